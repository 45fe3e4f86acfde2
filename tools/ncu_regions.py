"""Contiguous equal-execution-count SASS regions of an ncu capture, by share of instructions.
python tools/ncu_regions.py <rep> [top]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
h, d = rows[1], rows[2:]
iE, iS = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
ex = [float(r[iE] or 0) for r in d]
sm = [float(r[iS] or 0) for r in d]
k, out = 0, []
while k < len(d):
    j = k
    while j + 1 < len(d) and ex[j + 1] == ex[k]:
        j += 1
    out.append((ex[k] * (j - k + 1), k, j, ex[k], sum(sm[k:j + 1])))
    k = j + 1
tot, ts = sum(ex), sum(sm)
for w, a, b, e, s in sorted(out, reverse=True)[:top]:
    print(f"{100*w/tot:5.1f}% instr {100*s/ts:5.1f}% stalls [{a}-{b}] n={b-a+1} ex={e:.0f} first: {d[a][1].strip()[:60]}")
