"""Triangular-solve timing (diagnostics): mf_precond_apply on a config's matrix, both schedules
(MF_SPTRSV_SWEEP=0/1) and recursive-block depths.  python tools/sptrsv_time.py [C4spd] [reps]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
name = sys.argv[1] if len(sys.argv) > 1 else "C4spd"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
only = os.environ.get("ONLY")
A = W.make(name)
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va)
r = torch.rand(A.n_rows, dtype=torch.float64, device="cuda")
for sweep in ("1", "0"):
    for rb in (0, 4):
        if only and only != f"{sweep}{rb}":
            continue
        os.environ["MF_SPTRSV_SWEEP"] = sweep
        P = mf.Precond(T, sptrsv=mf.SPTRSV_RECURSIVE_BLOCK, rb_depth=rb) if rb else mf.Precond(T)
        inf = P.info()
        z = P.apply(r)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(reps):
            z = P.apply(r)
        torch.cuda.synchronize()
        dt = (time.perf_counter() - t0) / reps
        print(f"{name} sweep={sweep} rb={rb}: {dt*1e3:.2f} ms per apply  depth_l={inf['depth_l']} depth_u={inf['depth_u']} "
              f"nnz_l={inf['nnz_l']} ns/row={dt*1e9/A.n_rows/2:.1f}", flush=True)
        P.close()
