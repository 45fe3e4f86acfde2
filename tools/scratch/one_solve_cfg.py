"""One conversion + solve with a given layout / block size (for ncu).  args: config layout B [mode]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
name, lay, B = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
mode = int(sys.argv[4]) if len(sys.argv) > 4 else 2
A = W.make(name)
b = torch.from_numpy(W.rhs_ones(A)).cuda()
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
fn = mf.cg_solve if W.CONFIGS[name]["solver"] == "cg" else mf.bicgstab_solve
for _ in range(2):
    T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va, layout=lay, block_threads=B)
    r = fn(T, b, max_iter=W.CONFIGS[name]["max_iter"], mode=mode, history=False)
    print(r.iterations, r.kernel_ms, flush=True)
