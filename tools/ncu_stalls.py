"""Stall-reason breakdown of an ncu capture, overall and for SASS index ranges.
python tools/ncu_stalls.py <rep> [a-b ...]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
h, d = rows[1], rows[2:]
cols = [k for k, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
def show(name, rng):
    tot = {h[k]: sum(float(d[i][k] or 0) for i in rng) for k in cols}
    s = sum(tot.values()) or 1
    print(f"{name}: samples {s:.0f}  " + "  ".join(f"{k[6:]} {100*v/s:.0f}%" for k, v in sorted(tot.items(), key=lambda kv: -kv[1]) if v / s > 0.02))
show("all", range(len(d)))
for a in sys.argv[2:]:
    lo, hi = map(int, a.split("-"))
    show(a, range(lo, hi + 1))
