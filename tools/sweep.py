"""Launch-shape sweep with the per-phase breakdown (diagnostic).  python tools/sweep.py C2 [max_iter]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
name = sys.argv[1] if len(sys.argv) > 1 else "C2"
max_iter = int(sys.argv[2]) if len(sys.argv) > 2 else W.CONFIGS[name]["max_iter"]
shapes = [(int(a), int(b)) for a, b in (x.split("x") for x in sys.argv[3].split(","))] if len(sys.argv) > 3 else \
    [(0, 256), (0, 512), (0, 1024), (296, 256)]
A = W.make(name)
b = torch.from_numpy(W.rhs_ones(A)).cuda()
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
fn = mf.cg_solve if W.CONFIGS[name]["solver"] == "cg" else mf.bicgstab_solve
names = {"cg": ["wait", "spmv", "red_sig", "upd_xr", "red_rr", "upd_p", "init"],
         "bicgstab": ["wait_p", "spmv_mu", "red_eta", "upd_s", "wait_s", "spmv_th", "red_tt", "upd_xr", "red_rho", "upd_p", "init"]}[W.CONFIGS[name]["solver"]]
layouts = [int(x) for x in sys.argv[4].split(",")] if len(sys.argv) > 4 else [0]
for (G, B), lay in [(sh, l) for sh in shapes for l in layouts]:
    for mode in (mf.MODE_DYNAMIC, mf.MODE_STATIC):
        try:
            T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va, grid_ctas=G, block_threads=B, layout=lay)
            kw = dict(cg_variant=int(os.environ.get("CGV", "0"))) if fn is mf.cg_solve else {}
            st = fn(T, b, max_iter=max_iter, mode=mode, collect_stats=True, history=False, raise_on_breakdown=False, **kw)
            r = fn(T, b, max_iter=max_iter, mode=mode, history=False, raise_on_breakdown=False, **kw)
        except mf.MFError as e:
            print(G, B, "error", e); continue
        it = max(r.iterations, 1)
        ph = " ".join(f"{n}={v/it*1e3:.1f}" for n, v in zip(names, r.phase_ms))
        print(f"{name} L={T.info()['layout']} G={T.info()['plan_G']} B={B} mode={mode}: it={r.iterations} conv={r.converged} {r.kernel_ms:.2f} ms "
              f"{r.kernel_ms/it*1e3:.1f} us/it  {st.model_bytes/r.kernel_ms/1e6:.0f} GB/s  barrier={r.barrier_ms/it*1e3:.1f} us/it | {ph}", flush=True)
        T.close()
