"""Row-block multi-GPU path (paper_conf_sc_yangznjs0t024_b200/dist.py).

CPU (-m "not gpu"): the partition / halo plan, and the distributed CG driver itself with
world_size 2 over gloo, its per-rank arithmetic supplied by a numpy test engine (tests only --
the product engine is libmf's CUDA kernels and has no CPU fallback).
GPU: with one rank over NCCL the driver (libmf kernels + rank-order reductions) reproduces the
single-kernel mf_cg_solve bit for bit."""
import math
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


class NumpyEngine:
    """Test-only per-rank arithmetic (FP64, plain order) on CPU tensors."""

    def matrix(self, n_local, n_ext, rowptr, colidx, vals, classify=True):
        return sp.csr_matrix((vals, colidx, rowptr), shape=(n_local, n_ext))

    def vector(self, n):
        return torch.zeros(int(n), dtype=torch.float64)

    def spmv(self, M, xe, y, level):
        assert level is None
        y.copy_(torch.from_numpy(M @ xe.numpy()))

    def levels(self, v, th):
        raise AssertionError("static mode only")

    def dot(self, M, u, v):
        return float(np.dot(u.numpy(), v.numpy()))

    def update_xr(self, M, alpha, p, mu, x, r):
        x.add_(alpha * p)
        r.sub_(alpha * mu)
        return float(torch.dot(r, r))

    def update_p(self, M, beta, r, p):
        p.mul_(beta).add_(r)


def plain_cg(A, b, tol=1e-10, max_iter=1000):
    M = sp.csr_matrix((A.vals, A.colidx, A.rowptr), shape=(A.n_rows, A.n_cols))
    x = np.zeros_like(b)
    r = b.copy()
    p = r.copy()
    rho = r @ r
    nb = math.sqrt(b @ b)
    j = 0
    while math.sqrt(rho) / nb >= tol and j < max_iter:
        mu = M @ p
        alpha = rho / (mu @ p)
        x += alpha * p
        r -= alpha * mu
        rr = r @ r
        p = r + (rr / rho) * p
        rho = rr
        j += 1
    return x, j


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
    """3D 7-point Poisson 32^3 in 4 slabs: each interior rank exchanges exactly one 32x32 plane
    with each neighbour (the C5 pattern)."""
    m = 32
    A = W.poisson3d(m)
    P = 4
    bnd = dist.partition_rows(A.n_rows, P)
    ext = []
    for k in range(P):
        rp, ci, _ = dist.local_rows(A, bnd[k], bnd[k + 1])
        ext.append((bnd[k], bnd[k + 1]) + dist.local_extent(ci, bnd[k], bnd[k + 1], A.n_rows))
    plans = [dist.HaloPlan.build(k, ext) for k in range(P)]
    plane = m * m
    for k, pl in enumerate(plans):
        peers = sorted(q for q, _, _ in pl.recv)
        assert peers == [q for q in (k - 1, k + 1) if 0 <= q < P]
        assert all(hi - lo == plane for _, lo, hi in pl.recv)
        # what k receives from q is exactly what q sends to k
        for q, lo, hi in pl.recv:
            assert (k, lo, hi) in plans[q].send


def _worker(rank, world, port, out):
    import torch.distributed as td
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    td.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.poisson3d(16)
        b = W.rhs_ones(A)
        bnd = dist.partition_rows(A.n_rows, world, A.rowptr)
        rb, re = bnd[rank], bnd[rank + 1]
        comm = dist.Comm()
        D = dist.DistMatrix(NumpyEngine(), comm, A.n_rows, rb, re, *dist.local_rows(A, rb, re))
        res = dist.cg_solve(D, torch.from_numpy(b[rb:re].copy()), mode="static")
        xs = [torch.zeros(bnd[q + 1] - bnd[q], dtype=torch.float64) for q in range(world)]
        td.all_gather(xs, res.x)
        if rank == 0:
            np.save(out, np.concatenate([t.numpy() for t in xs]))
            np.save(out + ".it.npy", np.array([res.iterations, int(res.converged), res.halo_bytes]))
    finally:
        td.destroy_process_group()


@pytest.mark.dist
def test_dist_cg_gloo_world2_matches_single_process(tmp_path):
    import torch.multiprocessing as tmp
    out = str(tmp_path / "x.npy")
    tmp.spawn(_worker, args=(2, free_port(), out), nprocs=2, join=True)
    x = np.load(out)
    it, conv, halo = np.load(out + ".it.npy")
    A = W.poisson3d(16)
    b = W.rhs_ones(A)
    xr, jr = plain_cg(A, b)
    assert conv == 1 and abs(int(it) - jr) <= 1
    assert np.linalg.norm(x - xr) / np.linalg.norm(xr) < 1e-8
    assert np.max(np.abs(x - 1.0)) < 1e-6          # b = A*1
    assert halo == 16 * 16 * 8 * int(it)           # one 16x16 plane per iteration from the neighbour


@pytest.mark.gpu
def test_dist_world1_bit_identical_to_single_kernel():
    """One rank over NCCL: the distributed driver equals mf_cg_solve bit for bit (histories, x)."""
    import torch.distributed as td
    import paper_conf_sc_yangznjs0t024_b200 as mf
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(free_port()))
    td.init_process_group("nccl", rank=0, world_size=1)
    try:
        for name, scale in (("C2", 16), ("C1", 64)):
            A = W.make(name, scale)
            b = W.rhs_ones(A)
            T = mf.TileMatrix.from_host_csr(A)
            ref = mf.cg_solve(T, torch.from_numpy(b).cuda(), mode=mf.MODE_DYNAMIC, tol=1e-10, max_iter=1000)
            D = dist.DistMatrix(dist.CudaEngine("cuda"), dist.Comm(), A.n_rows, 0, A.n_rows, *dist.local_rows(A, 0, A.n_rows))
            res = dist.cg_solve(D, torch.from_numpy(b).cuda(), tol=1e-10, max_iter=1000, mode="dynamic")
            assert res.converged and res.iterations == ref.iterations
            assert np.array_equal(res.history, ref.history)
            assert torch.equal(res.x, ref.x)
    finally:
        td.destroy_process_group()
