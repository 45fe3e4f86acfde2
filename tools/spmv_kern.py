"""Standalone SpMV kernel timing (diagnostics): MF_SPMV_REPS launches of the mf_spmv kernel on C2.
python tools/spmv_kern.py [C2] [dyn]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("MF_SPMV_REPS", "50")
import torch
import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
name = sys.argv[1] if len(sys.argv) > 1 else "C2"
A = W.make(name)
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va)
x = torch.rand(A.n_cols, dtype=torch.float64, device="cuda")
lev = torch.zeros((A.n_cols + 15) // 16, dtype=torch.uint8, device="cuda") if len(sys.argv) > 2 else None
T.spmv(x, lev)
torch.cuda.synchronize()
