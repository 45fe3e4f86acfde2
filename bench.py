#!/usr/bin/env python
"""Benchmark of the Mille-feuille hot path on B200 (BASELINE.json metric:
"CG/BiCGSTAB time-to-solution, iters/s; effective HBM GB/s vs B200 peak").

Workload (default): BASELINE.json configs[1] = C2, CG mixed precision (dynamic switch) on the
value-scaled 3D 7-point Poisson 128^3 (2,097,152 rows), b = A*1, x0 = 0, tol 1e-10.
A STEP is one pass of the whole hot path over the input: CSR (resident in HBM) -> tile
conversion + classification (mf_tile_matrix_from_csr) -> the single persistent CG kernel to
convergence (mf_cg_solve).  value = CG iterations per second over the timed steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl reference]

N > 1 (torchrun, one process per GPU): ONE solve of the config's matrix partitioned into row
blocks over the N GPUs (dist.py: NCCL halo exchange + rank-ordered scalar reductions; strong
scaling), timed on the device, max over ranks.
--impl reference: the oracle (oracle/, plain C, binary64) on the host cores, same metric and
config, each step a bounded sample of the workload (the first --ref-iters CG iterations).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "CG/BiCGSTAB time-to-solution, iters/s; effective HBM GB/s vs B200 peak"
UNIT = "iters/s"


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {"hbm_gbs": 6650.0, "_fallback": True}


def _config(name):
    import workloads as W
    spec = W.CONFIGS[name]
    desc = {"C1": "C1 (configs[0]): CG on 2D 5-point Poisson 64x64",
            "C2": "C2 (configs[1]): CG mixed precision on value-scaled 3D 7-point Poisson 128^3",
            "C3": "C3 (configs[2]): BiCGSTAB on 2D convection-diffusion 2048^2",
            "C5": "C5 (configs[4]): CG on 3D 7-point Poisson 512^3"}.get(name, spec["desc"])
    return spec, desc


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index=0):
        self.rows, self.proc, self.gpu = [], None, gpu_index

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([c.strip() for c in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows for k in range(4) if len(r) > 5 + k and r[5 + k] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def flush_l2(buf):
    buf.add_(1.0)     # 256 MiB write > 126 MB L2


def gpu_arm(args, rank, world):
    import torch

    import paper_conf_sc_yangznjs0t024_b200 as mf
    import workloads as W

    dev = torch.device("cuda", rank % max(torch.cuda.device_count(), 1))
    torch.cuda.set_device(dev)
    mf.build()
    mf.lib()
    spec, desc = _config(args.config)
    A = W.make(args.config)
    b_h = W.rhs_ones(A)
    solver = mf.cg_solve if spec["solver"] in ("cg", "pcg") else mf.bicgstab_solve
    max_iter = spec["max_iter"]
    stream = torch.cuda.current_stream()
    # inputs resident in HBM before the timed region
    rp = torch.from_numpy(A.rowptr).to(dev)
    ci = torch.from_numpy(A.colidx).to(dev)
    va = torch.from_numpy(A.vals).to(dev)
    b = torch.from_numpy(b_h).to(dev)
    flush = torch.empty(32 * 1024 * 1024, dtype=torch.float64, device=dev)

    def step():
        T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va)
        r = solver(T, b, max_iter=max_iter, mode=mf.MODE_DYNAMIC, history=False)
        return T, r

    # stats pass (untimed): exact per-SpMV effective precisions -> algorithmic bytes
    T0 = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va)
    stats = solver(T0, b, max_iter=max_iter, mode=mf.MODE_DYNAMIC, collect_stats=True, level_counts=True)
    info0 = T0.info()
    for _ in range(args.warmup):
        T, r = step()
        T.close()
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    evs = []
    iters, kern_ms, conv_ms = 0, [], []
    with Clocks(dev.index) as clk:
        torch.cuda.synchronize()
        for _ in range(args.steps):
            flush_l2(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            T, r = step()
            e1.record(stream)
            evs.append((e0, e1))
            iters += r.iterations
            kern_ms.append(r.kernel_ms)
            conv_ms.append(T.info()["convert_ms"])
            assert r.converged and r.iterations == stats.iterations, "non-deterministic or failed solve"
            T.close()
        torch.cuda.synchronize()
    step_ms = [a.elapsed_time(c) for a, c in evs]
    total_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        total_ms = float(t.item())
        it = torch.tensor([iters], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(it)
        iters_all = float(it.item())
    else:
        iters_all = float(iters)
    value = iters_all / (total_ms / 1e3)

    # end to end through the public API with host buffers (pinned), H2D + D2H inside
    rp_h = torch.from_numpy(A.rowptr).pin_memory()
    ci_h = torch.from_numpy(A.colidx).pin_memory()
    va_h = torch.from_numpy(A.vals).pin_memory()
    b_hh = torch.from_numpy(b_h).pin_memory()
    x_h = torch.empty(A.n_rows, dtype=torch.float64).pin_memory()
    e2e_ms, e2e_iters = 0.0, 0
    for k in range(args.warmup + args.steps):
        flush_l2(flush)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        rpd = rp_h.to(dev, non_blocking=True)
        cid = ci_h.to(dev, non_blocking=True)
        vad = va_h.to(dev, non_blocking=True)
        bd = b_hh.to(dev, non_blocking=True)
        T = mf.TileMatrix(A.n_rows, A.n_cols, rpd, cid, vad)
        r = solver(T, bd, max_iter=max_iter, mode=mf.MODE_DYNAMIC, history=False)
        x_h.copy_(r.x, non_blocking=True)
        e1.record(stream)
        torch.cuda.synchronize()
        if k >= args.warmup:
            e2e_ms += e0.elapsed_time(e1)
            e2e_iters += r.iterations
        T.close()
    h2d = A.rowptr.nbytes + A.colidx.nbytes + A.vals.nbytes + b_h.nbytes
    d2h = A.n_rows * 8

    peaks = _peaks()
    kms = statistics.mean(kern_ms)
    bytes_launch = stats.model_bytes          # algorithmic bytes of one solve launch (byte model)
    achieved = bytes_launch / (kms / 1e3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get(args.config, {}).get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    ntiles = info0["tilenum"]
    lc = stats.level_counts
    mix = (lc.sum(0) / max(lc.sum(), 1)).round(4).tolist() if lc is not None and lc.size else None
    line = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(total_ms / args.steps, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded workloads.py)",
        "config": {"workload": desc, "n": A.n_rows, "nnz": A.nnz, "tiles": ntiles, "solver": spec["solver"],
                   "mode": "dynamic mixed (FP64/FP32/FP16/E4M3 tiles + bypass)", "tol": 1e-10,
                   "step": "convert CSR->tiles + full solve", "l2": "flushed between steps (256 MiB write)",
                   "plan": {"G": info0["plan_G"], "B": info0["plan_B"]},
                   "parallelism": "weak: one independent instance per GPU" if world > 1 else "1 GPU"},
        "iterations": stats.iterations,
        "time_to_solution_ms": round(total_ms / args.steps, 4),
        "solve_kernel_ms": round(kms, 4),
        "convert_ms": round(statistics.mean(conv_ms), 4),
        "solve_iters_per_s": round(stats.iterations / (kms / 1e3), 1),
        "effective_gbs": round(achieved, 1),
        "tile_level_mix": mix,
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                     "frac": round(achieved / peaks["hbm_gbs"], 4), "traffic": traffic,
                     "kernel": "cg_persistent (whole solve, one launch)",
                     "bytes_per_launch": bytes_launch,
                     "peak_source": "fallback" if peaks.get("_fallback") else "measured (MEASURED_PEAKS.json hbm_gbs)"},
        "e2e": {"value": round(e2e_iters / (e2e_ms / 1e3), 3), "unit": UNIT, "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": d2h},
        "gpu_launches": args.steps * (info0.get("convert_launches", 0) + 1),
        "clocks": clk.summary(),
    }
    return line


def dist_arm(args, rank, world):
    """N > 1: ONE solve of the config's matrix row-partitioned over the N GPUs (SURVEY 8(e),
    paper_conf_sc_yangznjs0t024_b200/dist.py): NCCL halo exchange of p + rank-ordered scalar
    reductions, per-rank work in libmf kernels.  Strong scaling: value = CG iterations per second
    of the distributed solve; a step = per-rank conversion of its rows + the solve."""
    import torch
    import torch.distributed as td

    import paper_conf_sc_yangznjs0t024_b200 as mf
    import workloads as W
    from paper_conf_sc_yangznjs0t024_b200 import dist

    dev = torch.device("cuda", rank % max(torch.cuda.device_count(), 1))
    torch.cuda.set_device(dev)
    mf.build()
    mf.lib()
    spec, desc = _config(args.config)
    if spec["solver"] != "cg":
        raise SystemExit("row-partitioned multi-GPU path: CG configs (C1, C2, C5)")
    A = W.make(args.config)
    b_h = W.rhs_ones(A)
    bnd = dist.partition_rows(A.n_rows, world, A.rowptr)
    rb, re = bnd[rank], bnd[rank + 1]
    rp, ci, va = dist.local_rows(A, rb, re)
    b = torch.from_numpy(b_h[rb:re].copy()).to(dev)
    comm = dist.Comm()
    eng = dist.CudaEngine(dev)

    def step():
        D = dist.DistMatrix(eng, comm, A.n_rows, rb, re, rp, ci, va)
        return D, dist.cg_solve(D, b, tol=1e-10, max_iter=spec["max_iter"], mode="dynamic")

    for _ in range(args.warmup):
        D, r = step()
        conv_launches = D.M.info()["convert_launches"]
        D.M.close()
    torch.cuda.synchronize()
    td.barrier()
    stream = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(dev.index) as clk:
        torch.cuda.synchronize()
        e0.record(stream)
        iters = 0
        for _ in range(args.steps):
            D, r = step()
            assert r.converged
            iters += r.iterations
            D.M.close()
        e1.record(stream)
        torch.cuda.synchronize()
    ms = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
    td.all_reduce(ms, op=td.ReduceOp.MAX)
    total_ms = float(ms.item())
    value = iters / (total_ms / 1e3)
    # e2e through the public API with host inputs: this rank's CSR rows and b slice (host) ->
    # device inside the timed region, conversion + solve, x back to pinned host memory
    bh = torch.from_numpy(b_h[rb:re].copy()).pin_memory()
    xh = torch.empty(re - rb, dtype=torch.float64).pin_memory()
    td.barrier()
    torch.cuda.synchronize()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    e2e_it = 0
    for _ in range(args.steps):
        bd = bh.to(dev, non_blocking=True)
        D = dist.DistMatrix(eng, comm, A.n_rows, rb, re, rp, ci, va)
        r = dist.cg_solve(D, bd, tol=1e-10, max_iter=spec["max_iter"], mode="dynamic")
        xh.copy_(r.x, non_blocking=True)
        e2e_it += r.iterations
        D.M.close()
    f1.record(stream)
    torch.cuda.synchronize()
    ms2 = torch.tensor([f0.elapsed_time(f1)], dtype=torch.float64, device=dev)
    td.all_reduce(ms2, op=td.ReduceOp.MAX)
    peaks = _peaks()
    n = A.n_rows
    # byte model per iteration (global, all ranks): static TilePrec bytes + 48n vectors + halo planes
    line = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(total_ms / args.steps, 4), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded workloads.py)",
        "config": {"workload": desc, "n": n, "nnz": A.nnz, "solver": "cg", "tol": 1e-10,
                   "mode": "dynamic mixed (FP64/FP32/FP16/E4M3 tiles + bypass)",
                   "step": "per-rank conversion of its rows + one distributed solve",
                   "parallelism": f"row blocks over {world} GPUs (NCCL halo of p + rank-ordered scalar all-gathers)",
                   "partition_rows": bnd, "l2": "inputs larger than L2 per step (whole solve)"},
        "iterations": r.iterations,
        "halo_bytes_per_iteration_rank0": D.plan.bytes_per_exchange(),
        "e2e": {"value": round(e2e_it / (float(ms2.item()) / 1e3), 3), "unit": UNIT,
                "h2d_bytes_per_step": int(rp.nbytes + ci.nbytes + va.nbytes + 8 * (re - rb)),
                "d2h_bytes_per_step": int(8 * (re - rb))},
        # libmf kernels per step on this rank: conversion, 2 init dots (2 kernels each), and per
        # iteration levels + SpMV + dot (2) + fused x/r update (2) + p update
        "gpu_launches": int(args.steps * (conv_launches + 4 + 7 * r.iterations)),
        "clocks": clk.summary(),
    }
    return line


def cpu_baseline(args, sample_iters):
    import oracle
    import workloads as W
    spec, desc = _config(args.config)
    A = W.make(args.config)
    b = W.rhs_ones(A)
    T = oracle.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
    solve = oracle.cg if spec["solver"] in ("cg", "pcg") else oracle.bicgstab
    t0 = time.perf_counter()
    r = solve(T, b, mode=oracle.MODE_DYNAMIC, max_iter=sample_iters, tol=0.0)
    dt = time.perf_counter() - t0
    return {"value": round(r["iterations"] / dt, 4), "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"first {r['iterations']} iterations of the oracle's dynamic mixed-precision "
                      f"{spec['solver'].upper()} emulation on the full {args.config} matrix "
                      f"(plain C, single thread, {dt:.1f} s)"}


def reference_arm(args):
    import oracle
    import workloads as W
    spec, desc = _config(args.config)
    A = W.make(args.config)
    b = W.rhs_ones(A)
    solve = oracle.cg if spec["solver"] in ("cg", "pcg") else oracle.bicgstab
    times, its = [], 0
    for k in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        T = oracle.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
        r = solve(T, b, mode=oracle.MODE_DYNAMIC, max_iter=args.ref_iters, tol=0.0)
        dt = time.perf_counter() - t0
        if k >= args.warmup:
            times.append(dt)
            its += r["iterations"]
    total = sum(times)
    value = its / total
    sample = (f"each step: oracle conversion + the first {args.ref_iters} iterations of the dynamic "
              f"mixed-precision {spec['solver'].upper()} emulation on the full {args.config} matrix")
    return {"impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(total / args.steps * 1e3, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (seeded workloads.py)",
            "config": {"workload": desc, "n": A.n_rows, "nnz": A.nnz, "solver": spec["solver"]},
            "cpu_baseline": {"value": round(value, 4), "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": round(value, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def torch_dist_ready():
    import torch.distributed as td
    return td.is_available() and td.is_initialized()


def init_single_rank_group():
    """--dist with one process: a one-rank NCCL group (exercises the multi-GPU path on 1 GPU)."""
    import socket

    import torch
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", str(port))
    torch.distributed.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2", choices=["C1", "C2", "C3", "C5"])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-iters", type=int, default=12, help="oracle iterations per reference step")
    ap.add_argument("--cpu-sample-iters", type=int, default=100)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--dist", action="store_true", help="row-partitioned multi-GPU path even with one rank")
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        if rank == 0:
            print(json.dumps(reference_arm(args)), flush=True)
        return
    if world > 1:
        import torch
        torch.distributed.init_process_group("nccl", device_id=torch.device("cuda", int(os.environ.get("LOCAL_RANK", rank))))
    if world > 1 or args.dist:
        if not torch_dist_ready():
            init_single_rank_group()
        line = dist_arm(args, int(os.environ.get("LOCAL_RANK", rank)), world)
    else:
        line = gpu_arm(args, int(os.environ.get("LOCAL_RANK", rank)), world)
    if rank == 0:
        if world == 1 and not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(args, args.cpu_sample_iters)
        print(json.dumps(line), flush=True)
    if torch_dist_ready():
        import torch
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
