"""the single persistent kernel against the multi-kernel classic path (one kernel
per SpMV / reduction / vector update, the structure of the paper's cuSPARSE baseline)
on the C2 matrix family from 16^3 to 160^3 rows, 100 iterations each (tol = 0).

  python tools/f3_crossover.py [sizes]      (one GPU; prints one JSON line per size)

multi_eager: libmf's row-block path at one rank with MF_DIST_NO_GRAPH (every kernel launched from
the host, as a library-call baseline does); multi_graph: the same kernels replayed as a CUDA
graph; single: mf_cg_solve (one cooperative kernel, grid barriers).  barrier_share is the
single kernel's %globaltimer barrier wait over its runtime (the Fig. 2 analog on our side)."""
import json
import os
import socket
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import torch.distributed as td

import paper_conf_sc_yangznjs0t024_b200 as mf
import workloads as W
from paper_conf_sc_yangznjs0t024_b200 import dist


def main():
    sizes = [int(v) for v in sys.argv[1].split(",")] if len(sys.argv) > 1 else [16, 24, 32, 48, 64, 96, 128, 160]
    s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    td.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    comm = dist.Comm()
    its = 100
    for m in sizes:
        A = W.scaled_poisson3d(m, seed=1)
        b = torch.from_numpy(W.rhs_ones(A)).cuda()
        out = {"m": m, "n": A.n_rows, "nnz": int(A.nnz), "iterations": its}
        T = mf.TileMatrix.from_host_csr(A)
        for mode, key in ((mf.MODE_STATIC, "static"), (mf.MODE_DYNAMIC, "dynamic")):
            rs = [mf.cg_solve(T, b, tol=0.0, max_iter=its, mode=mode, history=False) for _ in range(3)]
            r = min(rs, key=lambda q: q.kernel_ms)
            out[f"single_{key}_us_per_it"] = r.kernel_ms / its * 1e3
            out[f"single_{key}_barrier_share"] = r.barrier_ms / r.kernel_ms
        T.close()
        D = dist.DistTileMatrix.from_host_csr(comm, A, 0, A.n_rows)
        for graph in (False, True):
            if graph:
                os.environ.pop("MF_DIST_NO_GRAPH", None)
            else:
                os.environ["MF_DIST_NO_GRAPH"] = "1"
            rs = [dist.cg_solve(D, b, tol=0.0, max_iter=its, mode=mf.MODE_STATIC, history=False) for _ in range(3)]
            r = min(rs, key=lambda q: q.kernel_ms)
            out["multi_graph_us_per_it" if graph else "multi_eager_us_per_it"] = r.kernel_ms / its * 1e3
        os.environ.pop("MF_DIST_NO_GRAPH", None)
        D.close()
        out["speedup_single_vs_eager"] = out["multi_eager_us_per_it"] / out["single_static_us_per_it"]
        out["speedup_single_vs_graph"] = out["multi_graph_us_per_it"] / out["single_static_us_per_it"]
        print(json.dumps(out), flush=True)
    comm.close()
    td.destroy_process_group()


if __name__ == "__main__":
    main()
