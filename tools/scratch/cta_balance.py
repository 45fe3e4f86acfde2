"""Per-CTA balance diagnostics for the persistent solve (needs MF_PHASE_DUMP=1 output on stdin)."""
import sys, re
import numpy as np
txt = sys.stdin.read()
sp = np.array([float(v) for v in re.search(r"spmv per CTA:(.*)", txt).group(1).split()])
rows = np.array([int(v) for v in re.search(r"rows per CTA:(.*)", txt).group(1).split()])
print("spmv ms per CTA: min %.2f mean %.2f max %.2f" % (sp.min(), sp.mean(), sp.max()))
print("rows per CTA: min %d max %d" % (rows.min(), rows.max()))
print("corr(spmv, rows) = %.3f" % np.corrcoef(sp, rows)[0, 1])
print("spmv by CTA index (16 per line):")
for k in range(0, len(sp), 16):
    print(" ".join("%5.1f" % v for v in sp[k:k + 16]))
import sys as _s
sys.path.insert(0, ".")
