"""C3 convergence across precision modes / plans (diagnostic)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 2048
A = W.make("C3", scale)
b = torch.from_numpy(W.rhs_ones(A)).cuda()
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
cases = [(0, 0, 0, None), (1, 1, 0, None), (1, 2, 0, None), (1, 2, 0, 1e-13), (1, 2, 0, 1e-14), (1, 2, 0, 1e-15)]
for classify, mode, G, eps in cases:
    T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va, classify=bool(classify), grid_ctas=G)
    t = time.time()
    r = mf.bicgstab_solve(T, b, max_iter=20000, mode=mode, switch_eps=eps, raise_on_breakdown=False, collect_stats=True)
    h = r.history
    print(f"classify={classify} mode={mode} G={T.info()['plan_G']} eps={eps}: it={r.iterations} conv={r.converged} st={r.status} "
          f"relres={r.rel_residual:.3e} min={np.nanmin(h):.3e} at {int(np.nanargmin(h))} {r.kernel_ms/ max(r.iterations,1)*1e3:.1f} us/it "
          f"GB/s={r.model_bytes/r.kernel_ms/1e6:.0f}", flush=True)
    T.close()
