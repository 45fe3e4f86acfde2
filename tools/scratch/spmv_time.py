"""Time the standalone SpMV (mf_spmv: the same device code as the solver's SpMV phase).
python tools/spmv_time.py C2 [block_threads]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
name = sys.argv[1] if len(sys.argv) > 1 else "C2"
B = int(sys.argv[2]) if len(sys.argv) > 2 else 512
A = W.make(name)
rp, ci, va = (torch.from_numpy(a).cuda() for a in (A.rowptr, A.colidx, A.vals))
x = torch.rand(A.n_cols, dtype=torch.float64, device="cuda")
lev = torch.zeros((A.n_cols + 15) // 16, dtype=torch.uint8, device="cuda")
y = torch.empty(A.n_rows, dtype=torch.float64, device="cuda")
T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va, block_threads=B)
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
    print(f"{name} dbg={os.environ.get('MF_PIPE_DBG', '0')} layout={inf['layout']} B={B} G={inf['plan_G']} dyn={lv is not None}: "
          f"{ms*1e3:.1f} us  kernel_bytes={inf.get('kernel_bytes', 0)/1e6:.1f} MB -> {inf.get('kernel_bytes', 0)/ms/1e6:.0f} GB/s", flush=True)
