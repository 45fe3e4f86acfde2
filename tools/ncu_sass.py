"""Per-SASS-instruction view of an ncu capture: executions, stall samples, opcode mix.
python tools/ncu_sass.py <rep> [top]"""
import csv, io, subprocess, sys, collections
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
h, data = rows[1], rows[2:]
iS, iE = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
ex = [float(r[iE] or 0) for r in data]
smp = [float(r[iS] or 0) for r in data]
print("# kernel:", rows[0][1][:120])
print(f"# executed warp-instructions {sum(ex):.4g}, stall samples {sum(smp):.4g}")
mix = collections.Counter()
for r, e in zip(data, ex):
    op = r[1].strip().split()
    op = [o for o in op if not o.startswith("@")]
    mix[op[0].split(".")[0] if op else "?"] += e
print("# opcode mix (share of executed):", ", ".join(f"{k} {100*v/sum(ex):.1f}%" for k, v in mix.most_common(18)))
print("# top by stall samples:")
for k in sorted(range(len(data)), key=lambda k: -smp[k])[:top]:
    print(f"{100*smp[k]/sum(smp):6.2f}% ex={ex[k]:>10.0f} [{k}] {data[k][1].strip()[:70]}")
