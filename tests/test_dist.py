"""Row-block multi-GPU path (libmf dist.cu through paper_conf_sc_yangznjs0t024_b200.dist).

CPU (-m "not gpu"): the row partition, and libmf's host halo planner (mf_dist_plan) driven by a
world-size-2 gloo job: each rank plans its halo with libmf, the ranks exchange their requests over
gloo exactly as dist_create does over NCCL, and a numpy emulation of the distributed SpMV built
from those plans (own segments + received halo segments, remapped columns) equals the global SpMV.
GPU: one rank over NCCL -- mf_cg_solve_dist / mf_bicgstab_solve_dist equal the oracle's
kernel-order emulation bit for bit (histories, x) and the single-kernel solves."""
import os
import socket

import numpy as np
import pytest
import scipy.sparse as sp
import torch

import workloads as W
from paper_conf_sc_yangznjs0t024_b200 import dist


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_partition_rows_tile_aligned_and_balanced():
    A = W.make("C2", 32)
    for P in (1, 2, 3, 4, 8):
        bnd = dist.partition_rows(A.n_rows, P, A.rowptr)
        assert bnd[0] == 0 and bnd[-1] == A.n_rows and len(bnd) == P + 1
        assert all(b % 16 == 0 for b in bnd[:-1]) and all(bnd[k] <= bnd[k + 1] for k in range(P))
        nnz = [A.rowptr[bnd[k + 1]] - A.rowptr[bnd[k]] for k in range(P)]
        tr_nnz = int(np.max(A.rowptr[16::16] - A.rowptr[:-16:16]))
        assert max(nnz) - min(nnz) <= 2 * (tr_nnz + 16)      # balanced to within a tile row per side


def test_halo_plan_slab_stencil():
    """3D 7-point Poisson 32^3 in 4 slabs (the C5 pattern): every interior rank receives exactly one
    32x32 plane (64 segments) from each neighbour and nothing else."""
    m = 32
    A = W.poisson3d(m)
    P = 4
    bnd = dist.partition_rows(A.n_rows, P)
    plane_segs = m * m // 16
    for k in range(P):
        _, ci, _ = dist.local_rows(A, bnd[k], bnd[k + 1])
        segs, counts = dist.halo_plan(A.n_rows, bnd, k, ci)
        want = np.zeros(P, np.int64)
        for q in (k - 1, k + 1):
            if 0 <= q < P:
                want[q] = plane_segs
        assert np.array_equal(counts, want)
        assert np.all(np.diff(segs) > 0) and len(segs) == want.sum()


def test_halo_plan_scattered_is_exact():
    """C4-shaped scattered pattern: the plan lists exactly the off-block segments the rows touch
    (no column hull), each attributed to its owner."""
    A = W.make("C4spd", 1 << 13)
    P = 3
    bnd = dist.partition_rows(A.n_rows, P, A.rowptr)
    for k in range(P):
        _, ci, _ = dist.local_rows(A, bnd[k], bnd[k + 1])
        segs, counts = dist.halo_plan(A.n_rows, bnd, k, ci)
        g = np.unique(ci.astype(np.int64) >> 4)
        own = (g >= bnd[k] // 16) & (g < (bnd[k + 1] + 15) // 16)
        assert np.array_equal(segs, g[~own])
        owner = np.searchsorted(np.asarray(bnd[1:]), segs.astype(np.int64) * 16, side="right")
        assert np.array_equal(np.bincount(owner, minlength=P), counts)


def _worker(rank, world, port, out):
    import torch.distributed as td
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    td.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.make("C4ind", 1 << 12)
        bnd = dist.partition_rows(A.n_rows, world, A.rowptr)
        rb, re = bnd[rank], bnd[rank + 1]
        rp, ci, va = dist.local_rows(A, rb, re)
        segs, counts = dist.halo_plan(A.n_rows, bnd, rank, ci)
        # requests: the segments I need from each peer (what dist_create sends over NCCL)
        cnt = torch.from_numpy(counts.copy())
        allc = [torch.zeros_like(cnt) for _ in range(world)]
        td.all_gather(allc, cnt)
        off = np.concatenate([[0], np.cumsum(counts)])
        reqs = {}
        for q in range(world):
            if q == rank:
                continue
            mine = torch.from_numpy(segs[off[q]:off[q + 1]].astype(np.int64))
            theirs = torch.zeros(int(allc[q][rank]), dtype=torch.int64)
            if rank < q:
                td.send(mine, q); td.recv(theirs, q)
            else:
                td.recv(theirs, q); td.send(mine, q)
            reqs[q] = theirs.numpy()
        # halo exchange of x (segments of 16) along the plans, then the local SpMV
        x = np.random.default_rng(7).standard_normal(A.n_rows)
        nown = (re - rb + 15) // 16
        xe = np.zeros((nown + len(segs)) * 16)
        xe[:re - rb] = x[rb:re]
        for q in range(world):
            if q == rank:
                continue
            send = np.concatenate([x[s * 16:s * 16 + 16] for s in reqs[q]]) if len(reqs[q]) else np.zeros(0)
            assert all(bnd[rank] <= s * 16 < bnd[rank + 1] for s in reqs[q])
            rbuf = torch.zeros(16 * int(counts[q]), dtype=torch.float64)
            if rank < q:
                td.send(torch.from_numpy(send), q); td.recv(rbuf, q)
            else:
                td.recv(rbuf, q); td.send(torch.from_numpy(send), q)
            xe[(nown + off[q]) * 16:(nown + off[q + 1]) * 16] = rbuf.numpy()
        pos = {int(s): k for k, s in enumerate(segs)}
        cl = np.array([c - rb if rb <= c < re else (nown + pos[c >> 4]) * 16 + (c & 15) for c in ci], np.int64)
        y = sp.csr_matrix((va, cl, rp), shape=(re - rb, len(xe))) @ xe
        yall = torch.zeros(A.n_rows, dtype=torch.float64)
        yall[rb:re] = torch.from_numpy(y)
        td.all_reduce(yall)                      # disjoint slices: the sum assembles y
        if rank == 0:
            np.save(out, yall.numpy())
    finally:
        td.destroy_process_group()


@pytest.mark.dist
def test_dist_plan_gloo_world2_spmv_exact(tmp_path):
    import torch.multiprocessing as tmp
    out = str(tmp_path / "y.npy")
    tmp.spawn(_worker, args=(2, free_port(), out), nprocs=2, join=True)
    A = W.make("C4ind", 1 << 12)
    x = np.random.default_rng(7).standard_normal(A.n_rows)
    yref = sp.csr_matrix((A.vals, A.colidx, A.rowptr), shape=(A.n_rows, A.n_cols)) @ x
    assert np.allclose(np.load(out), yref, rtol=1e-13, atol=1e-13)


@pytest.mark.gpu
def test_dist_world1_matches_oracle_and_single_kernel(orc):
    """One rank over NCCL: the distributed solves equal the oracle's kernel-order emulation bit for
    bit (histories and x), hence the single-kernel solves too."""
    import torch.distributed as td
    import paper_conf_sc_yangznjs0t024_b200 as mf
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(free_port()))
    td.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        comm = dist.Comm()
        for name, scale, solver in (("C2", 16, "cg"), ("C1", 64, "cg"), ("C3", 64, "bicgstab"), ("C4spd", 1 << 12, "cg")):
            A = W.make(name, scale)
            b = W.rhs_ones(A)
            D = dist.DistTileMatrix.from_host_csr(comm, A, 0, A.n_rows)
            assert D.dist_info()["halo_segments"] == 0
            g, bb, R = D.plan()
            T = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
            ofn = orc.cg if solver == "cg" else orc.bicgstab
            ro = ofn(T, b, mode=2, plan=orc.Plan(g, bb, R), max_iter=2000)
            fn = dist.cg_solve if solver == "cg" else dist.bicgstab_solve
            Ts = mf.TileMatrix.from_host_csr(A)
            sfn = mf.cg_solve if solver == "cg" else mf.bicgstab_solve
            rs = sfn(Ts, torch.from_numpy(b).cuda(), mode=mf.MODE_DYNAMIC, max_iter=2000)
            # CG: the device-initiated kernel (dist_mode 2) and the host-orchestrated path (1)
            for dm in ((2, 1) if solver == "cg" else (1,)):
                res = fn(D, torch.from_numpy(b).cuda(), mode=mf.MODE_DYNAMIC, max_iter=2000, dist_mode=dm)
                assert res.converged and ro["converged"] and res.iterations == ro["iterations"], (name, dm)
                assert np.array_equal(res.history, ro["history"]), (name, dm)
                assert np.array_equal(res.x.cpu().numpy(), ro["x"]), (name, dm)
                assert torch.equal(rs.x, res.x), (name, dm)
            if solver == "bicgstab":
                with pytest.raises(mf.MFError):
                    fn(D, torch.from_numpy(b).cuda(), dist_mode=2)
            Ts.close()
            D.close()
        comm.close()
    finally:
        td.destroy_process_group()


def _run_local_group(A, P, ctas, mode, max_iter, switch_eps=None):
    """P ranks in P threads of this process on cuda:0 (mf_local_group), device-initiated CG."""
    import threading
    import paper_conf_sc_yangznjs0t024_b200 as mf
    bnd = dist.partition_rows(A.n_rows, P, A.rowptr)
    b = W.rhs_ones(A)
    grp = dist.LocalGroup(P)
    out, err = [None] * P, []

    def job(k):
        try:
            torch.cuda.set_device(0)
            st = torch.cuda.Stream()
            with torch.cuda.stream(st):
                comm = grp.comm(k)
                D = dist.DistTileMatrix.from_host_csr(comm, A, bnd[k], bnd[k + 1], grid_ctas=ctas)
                plan = D.plan()
                bk = torch.from_numpy(np.ascontiguousarray(b[bnd[k]:bnd[k + 1]])).cuda()
                r = dist.cg_solve(D, bk, mode=mode, max_iter=max_iter, dist_mode=2, watchdog_ms=20000,
                                  switch_eps=switch_eps, raise_on_breakdown=False)
                out[k] = (plan, r.x.cpu().numpy(), r.history, r.iterations, r.converged, r.status, D.dist_info())
                D.close()
                comm.close()
        except Exception as e:   # re-raised in the main thread
            err.append(e)

    th = [threading.Thread(target=job, args=(k,)) for k in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    grp.close()
    if err:
        raise err[0]
    return bnd, out


def _rank_plan(orc, bnd, out):
    R, Gr = [], [0]
    B = out[0][0][1]
    for k, o in enumerate(out):
        g, bb, Rk = o[0]
        assert bb == B
        R.extend((np.asarray(Rk[:-1], np.int64) + bnd[k]).tolist())
        Gr.append(Gr[-1] + g)
    R.append(bnd[-1])
    return orc.Plan(Gr[-1], B, np.array(R, np.int64), rank_ctas=Gr)


LOCAL_CASES = [("C2", 24, 2, 8), ("C2", 24, 3, 6), ("C1", 64, 2, 4), ("C4spd", 1 << 13, 3, 8)]


@pytest.mark.gpu
@pytest.mark.parametrize("name,scale,P,ctas", LOCAL_CASES)
def test_local_group_device_initiated_matches_oracle(orc, name, scale, P, ctas):
    """P ranks emulated on one GPU run the device-initiated kernel (halo stores into the peers'
    windows, arrival counters, tagged rank partials): histories and x equal the oracle's emulation
    of the global matrix under the rank-partitioned plan, bit for bit, in dynamic and static mode."""
    import paper_conf_sc_yangznjs0t024_b200 as mf
    A = W.make(name, scale)
    b = W.rhs_ones(A)
    T = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
    for mode in (mf.MODE_DYNAMIC, mf.MODE_STATIC):
        bnd, out = _run_local_group(A, P, ctas, mode, 400)
        assert sum(o[6]["halo_segments"] for o in out) > 0          # the ranks really exchange
        plan = _rank_plan(orc, bnd, out)
        ro = orc.cg(T, b, mode=2 if mode == mf.MODE_DYNAMIC else 1, plan=plan, max_iter=400)
        x = np.concatenate([o[1] for o in out])
        for o in out:
            assert o[5] == 0 and o[3] == ro["iterations"] and o[4] == ro["converged"], (name, mode)
            assert np.array_equal(o[2], ro["history"]), (name, mode)
        assert np.array_equal(x, ro["x"]), (name, mode)
