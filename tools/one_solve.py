"""One conversion + one solve of a config (for ncu captures): python tools/one_solve.py C2 [reps]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_yangznjs0t024_b200 as mf  # noqa: E402
import workloads as W  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
mode = int(sys.argv[3]) if len(sys.argv) > 3 else mf.MODE_DYNAMIC
A = W.make(name)
b = torch.from_numpy(W.rhs_ones(A)).cuda()
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
spec = W.CONFIGS[name]
fn = mf.cg_solve if spec["solver"] == "cg" else mf.bicgstab_solve
for _ in range(reps):
    T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va)
    r = fn(T, b, max_iter=spec["max_iter"], mode=mode, history=False, switch_eps=spec.get("switch_eps"))
    print(name, r.iterations, r.converged, f"{r.kernel_ms:.3f} ms", T.info()["convert_ms"], flush=True)
    T.close()
