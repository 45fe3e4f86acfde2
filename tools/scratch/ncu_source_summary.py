"""Stall-sample breakdown of the persistent CG kernel from the SASS source page of a full ncu
capture (gpurun_out/prof_cg_dyn.ncu-rep): the top instructions and the share of the SpMV region vs
the vector/reduction region.  python tools/ncu_source_summary.py > profiles/r01_ncu_cg_source.txt"""
import csv
import io
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
rep = os.path.join(ROOT, "gpurun_out", "prof_cg_dyn.ncu-rep")
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
h, data = rows[1], rows[2:]
iS, iE = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
smp = [float(r[iS] or 0) for r in data]
tot = sum(smp)
print(f"# {rows[0][1]}")
print(f"# warp stall samples: {tot:.0f} over {len(data)} SASS instructions")
print("# top 20 instructions (share of all samples, executions, SASS; the sample lands on the")
print("# instruction AFTER the one the warp waits on, e.g. after BAR.SYNC / the mbarrier try-wait)")
prev = {k: data[k - 1][1].strip() if k else "" for k in range(len(data))}
for k in sorted(sorted(range(len(data)), key=lambda k: -smp[k])[:20]):
    print(f"{100 * smp[k] / tot:6.2f}%  {data[k][iE]:>10}  {data[k][1].strip()[:60]:60s} | after: {prev[k][:40]}")
# regions: the SpMV pipeline spans the instructions that run once per stage (execution count of
# the mbarrier try-wait), the rest is per iteration or per row
tw = [k for k in range(len(data)) if "SYNCS.PHASECHK" in data[k][1]]
print("# mbarrier try-wait (TMA stage not yet landed):",
      " ".join(f"{100 * (smp[k] + smp[k + 1]) / tot:.2f}%" for k in tw))
bars = [k for k in range(len(data)) if "BAR.SYNC" in data[k][1]]
print(f"# samples on the instruction after a BAR.SYNC (CTA barrier waits, incl. the grid barrier's): "
      f"{100 * sum(smp[k + 1] for k in bars) / tot:.2f}%")
