#!/usr/bin/env python
"""Benchmark of the Mille-feuille hot path on B200 (BASELINE.json metric:
"CG/BiCGSTAB time-to-solution, iters/s; effective HBM GB/s vs B200 peak").

Workload (default): BASELINE.json configs[1] = C2, CG mixed precision (dynamic switch) on the
value-scaled 3D 7-point Poisson 128^3 (2,097,152 rows), b = A*1, x0 = 0, tol 1e-10.
A STEP is one pass of the whole hot path over the input: CSR (resident in HBM) -> tile
conversion + classification (mf_tile_matrix_from_csr) -> the single persistent kernel to
convergence (mf_cg_solve / mf_bicgstab_solve).  For C4 (PCG / PBiCGSTAB with ILU(0)) the
tile matrix and the ILU(0) factors are built once (setup, reported) and a step is the solve.
value = iterations per second over the timed steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl reference]

N > 1 (one process per GPU; spawned with torch.distributed.run when WORLD_SIZE is unset): ONE
solve of the config's matrix partitioned into row blocks over the N GPUs through libmf's
multi-GPU ABI (mf_tile_matrix_from_csr_dist + mf_cg_solve_dist: NCCL halo exchange,
rank-ordered reductions, device-side scalars), each rank generating only its own rows (C5);
strong scaling, timed on the device, max over ranks.  --dist runs that path with one rank.
--impl reference: the oracle (oracle/, plain C, binary64) on the host cores, same metric and
config, each step a bounded sample of the workload.
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
CONFIGS = ["C1", "C2", "C3", "C4spd", "C4ind", "C5"]


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
            "C4spd": "C4 (configs[3]): PCG (ILU(0)) on SuiteSparse-shaped SPD, 2^20 rows",
            "C4ind": "C4 (configs[3]): PBiCGSTAB (ILU(0)) on SuiteSparse-shaped indefinite, 2^20 rows",
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


def _phase_names(solver, pre):
    if solver in ("cg", "pcg") and not pre:
        return ["wait", "spmv", "reduce_sigma", "update_r", "reduce_rr", "update_xp", "init"]
    if solver in ("cg", "pcg"):
        return ["wait", "spmv", "reduce_sigma", "update_xr", "reduce_rr", "ilu_apply", "reduce_rz", "update_p", "", "", "init"]
    if not pre:
        return ["wait_p", "spmv_mu", "reduce_eta", "update_s", "wait_s", "spmv_theta", "reduce_tt", "update_xr",
                "reduce_rho", "update_p", "init"]
    return ["ilu_p", "spmv_mu", "reduce_eta", "update_s", "ilu_s", "spmv_theta", "reduce_tt", "update_xr",
            "update_p", "", "init"]


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
    pre = spec["solver"] in ("pcg", "pbicgstab")
    solver = mf.cg_solve if spec["solver"] in ("cg", "pcg") else mf.bicgstab_solve
    max_iter = spec["max_iter"]
    eps = spec.get("switch_eps")
    stream = torch.cuda.current_stream()
    # inputs resident in HBM before the timed region
    rp = torch.from_numpy(A.rowptr).to(dev)
    ci = torch.from_numpy(A.colidx).to(dev)
    va = torch.from_numpy(A.vals).to(dev)
    b = torch.from_numpy(b_h).to(dev)
    flush = torch.empty(32 * 1024 * 1024, dtype=torch.float64, device=dev)

    setup_ms = None
    Tpre = Mpre = None
    if pre:
        t0 = time.perf_counter()
        Tpre = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va)
        Mpre = mf.Precond(Tpre)
        torch.cuda.synchronize()
        setup_ms = (time.perf_counter() - t0) * 1e3

    def step(mode=mf.MODE_DYNAMIC, classify=True, **kw):
        if pre:
            return Tpre, solver(Tpre, b, max_iter=max_iter, mode=mode, switch_eps=eps, history=False, M=Mpre, **kw)
        T = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va, classify=classify)
        return T, solver(T, b, max_iter=max_iter, mode=mode, switch_eps=eps, history=False, **kw)

    def close(T):
        if not pre:
            T.close()

    # stats pass (untimed): exact per-SpMV effective precisions -> algorithmic bytes
    T0, stats = step(collect_stats=True, level_counts=True)
    info0 = T0.info()
    for _ in range(args.warmup):
        T, r = step()
        close(T)
    torch.cuda.synchronize()
    evs, iters, kern_ms, conv_ms, bar_ms, phases = [], 0, [], [], [], []
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
            bar_ms.append(r.barrier_ms)
            phases.append(r.phase_ms)
            conv_ms.append(T.info()["convert_ms"])
            assert r.converged and r.iterations == stats.iterations, "non-deterministic or failed solve"
            close(T)
        torch.cuda.synchronize()
    step_ms = [a.elapsed_time(c) for a, c in evs]
    total_ms = sum(step_ms)
    value = iters / (total_ms / 1e3)

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
        bd = b_hh.to(dev, non_blocking=True)
        if pre:     # the factors stay resident (setup); the step moves b in and x out
            r = solver(Tpre, bd, max_iter=max_iter, mode=mf.MODE_DYNAMIC, switch_eps=eps, history=False, M=Mpre)
            T = None
        else:
            rpd = rp_h.to(dev, non_blocking=True)
            cid = ci_h.to(dev, non_blocking=True)
            vad = va_h.to(dev, non_blocking=True)
            T = mf.TileMatrix(A.n_rows, A.n_cols, rpd, cid, vad)
            r = solver(T, bd, max_iter=max_iter, mode=mf.MODE_DYNAMIC, switch_eps=eps, history=False)
        x_h.copy_(r.x, non_blocking=True)
        e1.record(stream)
        torch.cuda.synchronize()
        if k >= args.warmup:
            e2e_ms += e0.elapsed_time(e1)
            e2e_iters += r.iterations
        if T is not None:
            T.close()
    h2d = b_h.nbytes + (0 if pre else A.rowptr.nbytes + A.colidx.nbytes + A.vals.nbytes)
    d2h = A.n_rows * 8

    # precision modes (Fig. 11 analog): the same solve in all-FP64 / static mixed
    modes = {"dynamic": {"iterations": stats.iterations, "solve_ms": round(statistics.mean(kern_ms), 3),
                         "us_per_iter": round(statistics.mean(kern_ms) / max(stats.iterations, 1) * 1e3, 2)}}
    if not args.no_modes:
        for name, mode, cls in (("static", mf.MODE_STATIC, True), ("fp64", mf.MODE_FP64, False)):
            T, r = step(mode=mode, classify=cls) if not pre else (None, None)
            if pre:   # the FP64 twin needs its own FP64 tile matrix + factors
                Tm = mf.TileMatrix(A.n_rows, A.n_cols, rp, ci, va, classify=cls)
                Mm = mf.Precond(Tm)
                r = solver(Tm, b, max_iter=max_iter, mode=mode, history=False, M=Mm)
                Mm.close()
                Tm.close()
            modes[name] = {"iterations": r.iterations, "converged": r.converged, "solve_ms": round(r.kernel_ms, 3),
                           "us_per_iter": round(r.kernel_ms / max(r.iterations, 1) * 1e3, 2),
                           "iters_per_s": round(r.iterations / (r.kernel_ms / 1e3), 1)}
            if T is not None:
                close(T)
        modes["dynamic_vs_fp64_time_to_solution"] = round(modes["fp64"]["solve_ms"] / modes["dynamic"]["solve_ms"], 3)
        if not pre:
            # the paper-literal sticky downgrade (reading R9): iteration inflation against the
            # per-iteration switch (cf. Table II)
            T, r = step(mode=mf.MODE_DYNAMIC, sticky=1, raise_on_breakdown=False)
            modes["sticky"] = {"iterations": r.iterations, "converged": r.converged, "status": r.status,
                               "solve_ms": round(r.kernel_ms, 3),
                               "us_per_iter": round(r.kernel_ms / max(r.iterations, 1) * 1e3, 2),
                               "iterations_vs_dynamic": round(r.iterations / max(stats.iterations, 1), 4)}
            close(T)

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
    lc = stats.level_counts
    mix = (lc.sum(0) / max(lc.sum(), 1)).round(4).tolist() if lc is not None and lc.size else None
    tp_mix = (np.array(info0["tiles_per_prec"]) / max(info0["tilenum"], 1)).round(4).tolist()
    pn = _phase_names(spec["solver"], pre)
    ph = np.mean(np.array(phases), axis=0) / max(stats.iterations, 1) * 1e3
    phase_us = {pn[k]: round(float(ph[k]), 2) for k in range(min(len(pn), len(ph))) if pn[k]}
    it_ms = kms / max(stats.iterations, 1)
    line = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(total_ms / args.steps, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded workloads.py)",
        "config": {"workload": desc, "n": A.n_rows, "nnz": A.nnz, "tiles": info0["tilenum"], "solver": spec["solver"],
                   "mode": "dynamic mixed (FP64/FP32/FP16/E4M3 tiles + bypass)", "tol": 1e-10,
                   "switch_eps": eps if eps is not None else "tol",
                   "step": "solve with the prebuilt tile matrix + ILU(0) (setup reported)" if pre
                   else "convert CSR->tiles + full solve",
                   "l2": "flushed between steps (256 MiB write)",
                   "plan": {"G": info0["plan_G"], "B": info0["plan_B"], "layout": "tile-synchronous TMA" if info0["layout"] == 2 else "compact"},
                   "parallelism": "1 GPU"},
        "iterations": stats.iterations,
        "time_to_solution_ms": round(total_ms / args.steps, 4),
        "solve_kernel_ms": round(kms, 4),
        "convert_ms": round(statistics.mean(conv_ms), 4),
        "setup_ms": None if setup_ms is None else round(setup_ms, 2),
        "solve_iters_per_s": round(stats.iterations / (kms / 1e3), 1),
        "us_per_iter": round(it_ms * 1e3, 2),
        "effective_gbs": round(achieved, 1),
        "barrier_share": round(statistics.mean(bar_ms) / kms, 4),
        "phase_us_per_iter": phase_us,
        "precision": {"tile_prec_mix": tp_mix, "dynamic_level_mix": mix,
                      "nnz_prec_mix": [round(v / max(sum(info0["nval"]), 1), 4) for v in info0["nval"]]},
        "modes": modes,
        "memory": {"csr_bytes": info0["csr_bytes"], "canonical_bytes": info0["canonical_bytes"],
                   "kernel_bytes": info0["kernel_bytes"],
                   "canonical_vs_csr": round(info0["canonical_bytes"] / max(info0["csr_bytes"], 1), 4)},
        "preprocessing": {"convert_ms": round(statistics.mean(conv_ms), 4),
                          "convert_in_iterations": round(statistics.mean(conv_ms) / it_ms, 2),
                          "convert_launches": info0["convert_launches"]},
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                     "frac": round(achieved / peaks["hbm_gbs"], 4), "traffic": traffic,
                     "kernel": f"{'p' if pre else ''}{'cg' if spec['solver'] in ('cg', 'pcg') else 'bicgstab'}_persistent (whole solve, one launch)",
                     "bytes_per_launch": bytes_launch,
                     "peak_source": "fallback" if peaks.get("_fallback") else "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"},
        "e2e": {"value": round(e2e_iters / (e2e_ms / 1e3), 3), "unit": UNIT, "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": d2h},
        "gpu_launches": args.steps * ((0 if pre else info0.get("convert_launches", 0)) + 1),
        "clocks": clk.summary(),
    }
    if pre:
        Mpre.close()
        Tpre.close()
    return line


def _local_problem(name, rb, re, W):
    """This rank's rows (C5: generated for the slab only) + b = A*1 restricted to them."""
    if name == "C5":
        L = W.poisson3d_rows(512, rb, re)
        return L.rowptr, L.colidx, L.vals, W.rhs_ones(L)
    A = W.make(name)
    a0, a1 = int(A.rowptr[rb]), int(A.rowptr[re])
    L = W.CSR(re - rb, A.n_cols, A.rowptr[rb:re + 1] - a0, A.colidx[a0:a1], A.vals[a0:a1])
    return L.rowptr, L.colidx, L.vals, W.rhs_ones(L)


def dist_arm(args, rank, world):
    """Row-partitioned solve over the N GPUs through libmf's multi-GPU ABI.
    Strong scaling: value = iterations per second of the one distributed solve; a step = per-rank
    conversion of its rows + the solve."""
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
    if spec["solver"] not in ("cg", "bicgstab"):
        raise SystemExit("row-partitioned multi-GPU path: unpreconditioned configs (C1, C2, C3, C5)")
    n = 512 ** 3 if args.config == "C5" else W.make(args.config).n_rows
    if args.config == "C5":
        bnd = [min(((n * k // world) // 16) * 16, n) for k in range(world)] + [n]
    else:
        bnd = dist.partition_rows(n, world, W.make(args.config).rowptr)
    rb, re = bnd[rank], bnd[rank + 1]
    rp_h, ci_h, va_h, b_h = _local_problem(args.config, rb, re, W)
    rp, ci, va = (torch.from_numpy(a).to(dev) for a in (rp_h, ci_h, va_h))
    b = torch.from_numpy(b_h).to(dev)
    comm = dist.Comm()
    fn = dist.cg_solve if spec["solver"] == "cg" else dist.bicgstab_solve
    eps = spec.get("switch_eps")

    # execution: auto (the device-initiated single kernel per rank when every rank is in one NVLink
    # domain, else host-orchestrated).  If the first solve fails on any rank (watchdog, setup), all
    # ranks switch to the host-orchestrated path (dist_mode 1) and the line says so.
    sel = {"dist_mode": 0, "fallback": None}

    def step():
        D = dist.DistTileMatrix(comm, n, rb, re, rp, ci, va)
        return D, fn(D, b, max_iter=spec["max_iter"], mode=mf.MODE_DYNAMIC, switch_eps=eps, history=False,
                     dist_mode=sel["dist_mode"], watchdog_ms=30000)

    try:
        D, r = step()
        ok, why = int(bool(r.converged)), "not converged"
        D.close()
    except mf.MFError as e:
        ok, why = 0, str(e)[:200]
    flag = torch.tensor([ok], dtype=torch.int32, device=dev)
    td.all_reduce(flag, op=td.ReduceOp.MIN)
    if int(flag.item()) == 0:
        sel["dist_mode"], sel["fallback"] = 1, f"device-initiated kernel failed ({why}); host-orchestrated path"
    for _ in range(args.warmup):
        D, r = step()
        conv_launches = D.info()["convert_launches"]
        halo = D.dist_info()
        D.close()
    torch.cuda.synchronize()
    td.barrier()
    stream = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(dev.index) as clk:
        torch.cuda.synchronize()
        e0.record(stream)
        iters, kms = 0, []
        for _ in range(args.steps):
            D, r = step()
            assert r.converged
            iters += r.iterations
            kms.append(r.kernel_ms)
            D.close()
        e1.record(stream)
        torch.cuda.synchronize()
    ms = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
    td.all_reduce(ms, op=td.ReduceOp.MAX)
    total_ms = float(ms.item())
    value = iters / (total_ms / 1e3)
    # e2e: this rank's CSR rows and b slice from pinned host memory, x back, inside the region
    hp = [torch.from_numpy(a).pin_memory() for a in (rp_h, ci_h, va_h, b_h)]
    xh = torch.empty(re - rb, dtype=torch.float64).pin_memory()
    td.barrier()
    torch.cuda.synchronize()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    e2e_it = 0
    for _ in range(args.steps):
        rpd, cid, vad, bd = (t.to(dev, non_blocking=True) for t in hp)
        D = dist.DistTileMatrix(comm, n, rb, re, rpd, cid, vad)
        r = fn(D, bd, max_iter=spec["max_iter"], mode=mf.MODE_DYNAMIC, switch_eps=eps, history=False,
               dist_mode=sel["dist_mode"], watchdog_ms=30000)
        xh.copy_(r.x, non_blocking=True)
        e2e_it += r.iterations
        D.close()
    f1.record(stream)
    torch.cuda.synchronize()
    ms2 = torch.tensor([f0.elapsed_time(f1)], dtype=torch.float64, device=dev)
    td.all_reduce(ms2, op=td.ReduceOp.MAX)
    comm.close()
    line = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(total_ms / args.steps, 4), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded workloads.py)",
        "config": {"workload": desc, "n": n, "solver": spec["solver"], "tol": 1e-10,
                   "mode": "dynamic mixed (FP64/FP32/FP16/E4M3 tiles + bypass)",
                   "step": "per-rank conversion of its rows + one distributed solve",
                   "parallelism": f"row blocks over {world} GPUs (libmf: NCCL halo of the SpMV input + rank-ordered all-gathered partials)",
                   "partition_rows": bnd, "l2": "inputs larger than L2 per step (whole solve)",
                   "dist_mode": "auto (device-initiated when available)" if sel["fallback"] is None else sel["fallback"]},
        "iterations": r.iterations,
        "solve_kernel_ms_rank0": round(statistics.mean(kms), 3),
        "halo_segments_rank0": halo["halo_segments"], "halo_bytes_per_exchange_rank0": halo["halo_segments"] * 144,
        "e2e": {"value": round(e2e_it / (float(ms2.item()) / 1e3), 3), "unit": UNIT,
                "h2d_bytes_per_step": int(rp_h.nbytes + ci_h.nbytes + va_h.nbytes + b_h.nbytes),
                "d2h_bytes_per_step": int(8 * (re - rb))},
        # per iteration: pack + SpMV + 2 rank partials + 2 scalar kernels + 2 vector kernels + stop
        # (CG); conversion per step
        "gpu_launches": int(args.steps * (conv_launches + 8 + 9 * r.iterations)),
        "clocks": clk.summary(),
    }
    return line


def cpu_baseline(args):
    """the oracle's textbook binary64 CSR solver (CG / BiCGSTAB, ILU(0) for C4)
    with OpenMP over all host cores in the affinity mask, and on one core; a bounded sample: the
    first K iterations where the full solve would exceed ~20 s."""
    import oracle
    import workloads as W
    spec, desc = _config(args.config)
    A = W.make(args.config)
    b = W.rhs_ones(A)
    kind = "cg" if spec["solver"] in ("cg", "pcg") else "bicgstab"
    M = None
    if spec["solver"] in ("pcg", "pbicgstab"):
        M = oracle.ILU0(A.rowptr, A.colidx, A.vals)
    cores = len(os.sched_getaffinity(0))
    try:
        model = subprocess.run(["lscpu"], capture_output=True, text=True).stdout
        cpu = next((l.split(":", 1)[1].strip() for l in model.splitlines() if l.startswith("Model name")), "unknown")
    except Exception:
        cpu = "unknown"
    out = {}
    for threads in (cores, 1):
        t0 = time.perf_counter()
        probe = oracle.baseline_solve(kind, A.rowptr, A.colidx, A.vals, b, M=M, max_iter=5, tol=0.0, threads=threads)
        per_it = (time.perf_counter() - t0) / max(probe["iterations"], 1)
        budget = max(5, int(20.0 / max(per_it, 1e-6)))
        t0 = time.perf_counter()
        r = oracle.baseline_solve(kind, A.rowptr, A.colidx, A.vals, b, M=M, max_iter=min(spec["max_iter"], budget),
                                  threads=threads)
        dt = time.perf_counter() - t0
        out[threads] = (r, dt)
    r, dt = out[cores]
    r1, dt1 = out[1]
    full = r["converged"]
    return {"value": round(r["iterations"] / dt, 3), "unit": UNIT, "cores": r["threads"], "kind": "oracle",
            "cpu": cpu,
            "sample": (f"oracle textbook binary64 CSR {kind.upper()}{' + ILU(0)' if M is not None else ''} "
                       f"(OpenMP, {r['threads']} threads), {'full solve to 1e-10' if full else 'first ' + str(r['iterations']) + ' iterations'}"
                       f" of the full {args.config} matrix in {dt:.2f} s"),
            "time_to_solution_s": round(dt, 3) if full else None,
            "one_core": {"value": round(r1["iterations"] / dt1, 3), "iterations": r1["iterations"], "seconds": round(dt1, 2)}}


def reference_arm(args):
    import oracle
    import workloads as W
    spec, desc = _config(args.config)
    A = W.make(args.config)
    b = W.rhs_ones(A)
    solve = oracle.cg if spec["solver"] in ("cg", "pcg") else oracle.bicgstab
    M = None
    if spec["solver"] in ("pcg", "pbicgstab"):
        T0 = oracle.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
        rp, ci, sv = T0.stored_csr()
        M = oracle.ILU0(rp, ci, sv)
    times, its = [], 0
    for k in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        T = oracle.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
        r = solve(T, b, mode=oracle.MODE_DYNAMIC, max_iter=args.ref_iters, tol=0.0, M=M,
                  switch_eps=spec.get("switch_eps"))
        dt = time.perf_counter() - t0
        if k >= args.warmup:
            times.append(dt)
            its += r["iterations"]
    total = sum(times)
    value = its / total
    sample = (f"each step: oracle conversion + the first {args.ref_iters} iterations of the dynamic "
              f"mixed-precision {spec['solver'].upper()} emulation on the full {args.config} matrix (1 thread)")
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
    """--dist with one process: a one-rank group (the multi-GPU path on 1 GPU)."""
    import socket

    import torch
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", str(port))
    torch.distributed.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))


def spawn(args):
    """--gpus N > 1 without a launcher: run this script under torch.distributed.run, N ranks."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2", choices=CONFIGS)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-iters", type=int, default=12, help="oracle iterations per reference step")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-modes", action="store_true", help="skip the static / FP64 comparison solves")
    ap.add_argument("--dist", action="store_true", help="row-partitioned multi-GPU path even with one rank")
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        if rank == 0:
            print(json.dumps(reference_arm(args)), flush=True)
        return
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn(args))
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
            line["cpu_baseline"] = cpu_baseline(args)
        print(json.dumps(line), flush=True)
    if torch_dist_ready():
        import torch
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
