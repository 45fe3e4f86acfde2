"""Time the standalone windowed SpMV (mf_spmv, same device code as the solver) per layout / block size."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
name = sys.argv[1] if len(sys.argv) > 1 else "C2"
A = W.make(name)
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
x = torch.rand(A.n_cols, dtype=torch.float64, device="cuda")
lev = torch.zeros((A.n_cols + 15) // 16, dtype=torch.uint8, device="cuda")
y = torch.empty(A.n_rows, dtype=torch.float64, device="cuda")
for lay in (1, 2):
    for B in (256, 512, 1024):
        T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va, block_threads=B, layout=lay)
        inf = T.info()
        for lv in (None, lev):
            for _ in range(3):
                T.spmv(x, lv, out=y)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(20):
                T.spmv(x, lv, out=y)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / 20
            nbytes = sum(inf["nval"][q] * [8, 4, 2, 1][q] for q in range(4)) + 2 * inf["slots"] + 16 * A.n_rows
            print(f"{name} layout={inf['layout']} B={B} G={inf['plan_G']} dyn={lv is not None}: {ms*1e3:.1f} us  "
                  f"~{nbytes/ms/1e6:.0f} GB/s (values+index+x+y)", flush=True)
        T.close()
