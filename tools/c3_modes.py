"""C3 (BiCGSTAB, convection-diffusion) across precision modes and switch thresholds: iterations,
convergence, true residual (the record behind workloads.CONFIGS["C3"]["switch_eps"]).
python tools/c3_modes.py [grid m]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 2048
A = W.make("C3", scale)
bh = W.rhs_ones(A)
b = torch.from_numpy(bh).cuda()
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
cases = [("fp64", 0, 0, None), ("static", 1, 1, None), ("dyn eps=tol", 1, 2, None), ("dyn eps=1e-11", 1, 2, 1e-11),
         ("dyn eps=1e-12", 1, 2, 1e-12), ("dyn eps=1e-13", 1, 2, 1e-13), ("dyn eps=1e-14", 1, 2, 1e-14),
         ("dyn eps=1e-15", 1, 2, 1e-15)]
for name, classify, mode, eps in cases:
    T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va, classify=bool(classify))
    r = mf.bicgstab_solve(T, b, max_iter=20000, mode=mode, switch_eps=eps, raise_on_breakdown=False, collect_stats=True,
                          level_counts=True)
    x = r.x.cpu().numpy()
    d = A.dense() if A.n_rows <= 4096 else None
    rows = np.repeat(np.arange(A.n_rows), np.diff(A.rowptr))
    ax = np.bincount(rows, weights=A.vals * x[A.colidx], minlength=A.n_rows)
    true_rel = float(np.linalg.norm(bh - ax) / np.linalg.norm(bh))
    lc = r.level_counts
    changed = float(np.mean(lc[:, 4] > 0)) if lc is not None and lc.size else 0.0
    print(f"{name:14s}: it={r.iterations} conv={r.converged} status={r.status} relres={r.rel_residual:.2e} "
          f"true={true_rel:.2e} |x-1|max={np.max(np.abs(x - 1)):.1e} {r.kernel_ms / max(r.iterations, 1) * 1e3:.1f} us/it "
          f"bypass-SpMVs={changed:.2f}", flush=True)
    T.close()
