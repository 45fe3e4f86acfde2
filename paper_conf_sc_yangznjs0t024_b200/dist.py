"""Row-block multi-GPU CG over NCCL (the paper's solver is single-GPU).

One process per GPU.  Rank k owns the tile-aligned rows [row_begin, row_end) of the global
matrix (contiguous blocks of 16-row tile rows, balanced on nonzeros).  Its rows gather the
contiguous column range [xlo, xhi) (rounded to 16-element segments, so local and global
segments -- and therefore tiles, TilePrec and the dynamic levels of Alg. 4 -- coincide); the
rank converts its rows as an n_local x (xhi - xlo) tile matrix and keeps the search direction
in an extended vector xe = p[xlo:xhi] whose own part is p[row_begin:row_end].

Per CG iteration (Alg. 1) on every rank:
  1. halo exchange: the slices of xe owned by other ranks are received over NCCL point-to-point
     (the owners send the rows each neighbour's tiles gather; for a 7-point stencil slab
     partition: one plane from each neighbour);
  2. levels of every segment of xe (Alg. 4) -> local SpMV mu = A~ xe (Alg. 5), libmf kernels;
  3. sigma = (mu, p): per-rank plan-tree partial, all-gathered, summed in rank order;
  4. x += alpha p, r -= alpha mu and (r, r) in one kernel; (r, r) all-gathered likewise;
  5. p = r + beta p (own rows) in a kernel.
Every arithmetic step runs in libmf's CUDA kernels (CudaEngine); this module only partitions,
plans and moves data (torch.distributed is the plumbing).  The reductions are deterministic:
the same inputs give the same bits on every rank and every run, and with one rank the solve
is bit-identical to the single-kernel mf_cg_solve (same plan tree, same operations).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

TS = 16


# ------------------------------------------------------------------ partition and halo plan
def partition_rows(n: int, nranks: int, rowptr=None) -> list[int]:
    """Row boundaries [0, r_1, ..., n] of nranks contiguous blocks of whole 16-row tile rows,
    balanced on (nonzeros + rows) per tile row."""
    ntr = (n + TS - 1) // TS
    tr_rows = np.full(ntr, TS, np.int64)
    if ntr:
        tr_rows[-1] = n - (ntr - 1) * TS
    if rowptr is not None:
        ends = np.minimum((np.arange(ntr, dtype=np.int64) + 1) * TS, n)
        starts = np.arange(ntr, dtype=np.int64) * TS
        cost = np.asarray(rowptr)[ends] - np.asarray(rowptr)[starts] + tr_rows
    else:
        cost = tr_rows
    pre = np.concatenate([[0], np.cumsum(cost)])
    tb = [0]                                   # boundaries in tile rows
    for k in range(1, nranks):
        t = int(np.searchsorted(pre, pre[-1] * k / nranks, side="left"))
        tb.append(min(max(t, tb[-1]), ntr))
    return [min(t * TS, n) for t in tb] + [n]


def local_extent(colidx, row_begin: int, row_end: int, n: int) -> tuple[int, int]:
    """[xlo, xhi): the 16-aligned column hull of this rank's rows and own range."""
    lo, hi = row_begin, row_end
    if len(colidx):
        lo = min(lo, int(np.min(colidx)))
        hi = max(hi, int(np.max(colidx)) + 1)
    lo = (lo // TS) * TS
    hi = min(((hi + TS - 1) // TS) * TS, n)
    return lo, hi


@dataclass
class HaloPlan:
    """recv[(peer, lo, hi)]: global rows of peer that land in my xe; send[(peer, lo, hi)]: my rows
    that peer's xe needs.  Derived from every rank's (row_begin, row_end, xlo, xhi)."""
    rank: int
    recv: list = field(default_factory=list)
    send: list = field(default_factory=list)

    @staticmethod
    def build(rank: int, ext: list[tuple[int, int, int, int]]) -> "HaloPlan":
        rb, re, xlo, xhi = ext[rank]
        plan = HaloPlan(rank)
        for q, (qb, qe, qlo, qhi) in enumerate(ext):
            if q == rank:
                continue
            lo, hi = max(xlo, qb), min(xhi, qe)          # q's rows inside my column hull
            if hi > lo:
                plan.recv.append((q, lo, hi))
            lo, hi = max(qlo, rb), min(qhi, re)          # my rows inside q's column hull
            if hi > lo:
                plan.send.append((q, lo, hi))
        return plan

    def bytes_per_exchange(self) -> int:
        return 8 * sum(hi - lo for _, lo, hi in self.recv)


def local_rows(A, row_begin: int, row_end: int):
    """Rows [row_begin, row_end) of a host CSR (global column ids): (rowptr, colidx, vals)."""
    a, b = int(A.rowptr[row_begin]), int(A.rowptr[row_end])
    return (np.ascontiguousarray(A.rowptr[row_begin:row_end + 1] - a), np.ascontiguousarray(A.colidx[a:b]),
            np.ascontiguousarray(A.vals[a:b]))


# ------------------------------------------------------------------ the compute engine (libmf)
class CudaEngine:
    """The product engine: every step in libmf's sm_100a kernels.  No fallback: a missing
    libmf.so or GPU raises MFError."""

    def __init__(self, device):
        import torch

        from . import lib
        lib()
        self.torch = torch
        self.device = torch.device(device)

    def matrix(self, n_local, n_ext, rowptr, colidx, vals, classify=True):
        from . import TileMatrix
        t = self.torch
        return TileMatrix(n_local, n_ext, t.from_numpy(rowptr).to(self.device), t.from_numpy(colidx).to(self.device),
                          t.from_numpy(vals).to(self.device), classify=classify)

    def vector(self, n):
        return self.torch.zeros(int(n), dtype=self.torch.float64, device=self.device)

    def spmv(self, M, xe, y, level):
        M.spmv(xe, level, out=y)

    def levels(self, v, th):
        from . import levels
        return levels(v, th)

    def dot(self, M, u, v) -> float:
        return M.dot(u, v)

    def update_xr(self, M, alpha, p, mu, x, r) -> float:
        return M.cg_update_xr(alpha, p, mu, x, r)

    def update_p(self, M, beta, r, p):
        M.cg_update_p(beta, r, p)


# ------------------------------------------------------------------ communication
class Comm:
    """torch.distributed plumbing: halo exchange and rank-ordered scalar sums."""

    def __init__(self, group=None):
        import torch
        import torch.distributed as td
        self.td, self.torch, self.group = td, torch, group
        self.size = td.get_world_size(group)
        self.rank = td.get_rank(group)
        self.backend = td.get_backend(group)

    def allgather_ints(self, vals, device):
        t = self.torch.tensor(vals, dtype=self.torch.int64, device=device)
        out = self.torch.empty(self.size * len(vals), dtype=self.torch.int64, device=device)
        self.td.all_gather_into_tensor(out, t, group=self.group)
        return out.cpu().numpy().reshape(self.size, len(vals)).tolist()

    def allsum(self, vals, device) -> list[float]:
        """Deterministic sum over ranks: all-gather the per-rank partials, add them in rank order."""
        if self.size == 1:
            return [float(v) for v in vals]
        t = self.torch.tensor(vals, dtype=self.torch.float64, device=device)
        out = self.torch.empty(self.size * len(vals), dtype=self.torch.float64, device=device)
        self.td.all_gather_into_tensor(out, t, group=self.group)
        g = out.cpu().numpy().reshape(self.size, len(vals))
        res = []
        for k in range(len(vals)):
            s = 0.0
            for q in range(self.size):
                s = s + float(g[q, k])
            res.append(s)
        return res

    def halo(self, xe, xlo: int, plan: HaloPlan):
        ops = []
        for q, lo, hi in plan.recv:
            ops.append(self.td.irecv(xe[lo - xlo:hi - xlo], src=self._g(q), group=self.group))
        for q, lo, hi in plan.send:
            ops.append(self.td.isend(xe[lo - xlo:hi - xlo], dst=self._g(q), group=self.group))
        for w in ops:
            w.wait()

    def _g(self, q):
        return q if self.group is None else self.td.get_global_rank(self.group, q)


# ------------------------------------------------------------------ the solve
@dataclass
class DistResult:
    x: object
    iterations: int
    converged: bool
    rel_residual: float
    history: np.ndarray
    status: str = "ok"
    halo_bytes: int = 0
    row_begin: int = 0
    row_end: int = 0


class DistMatrix:
    """This rank's rows of an n x n matrix, converted with the column hull [xlo, xhi)."""

    def __init__(self, engine, comm: Comm, n: int, row_begin: int, row_end: int, rowptr, colidx, vals, classify=True,
                 device=None):
        self.engine, self.comm, self.n = engine, comm, n
        self.row_begin, self.row_end = row_begin, row_end
        self.xlo, self.xhi = local_extent(colidx, row_begin, row_end, n)
        loc = (np.asarray(colidx, np.int64) - self.xlo).astype(np.int32)
        self.M = engine.matrix(row_end - row_begin, self.xhi - self.xlo, np.asarray(rowptr, np.int64), loc,
                               np.asarray(vals, np.float64), classify=classify)
        dev = device if device is not None else getattr(engine, "device", "cpu")
        self.comm_device = dev if comm.backend == "nccl" else "cpu"
        ext = comm.allgather_ints([row_begin, row_end, self.xlo, self.xhi], self.comm_device)
        self.plan = HaloPlan.build(comm.rank, [tuple(e) for e in ext])


def thresholds(switch_eps: float, v0norm: float, n: int, absolute: bool = False):
    """Alg. 4 thresholds with reading R8: tau = eps * ||v0||_2."""
    tau = switch_eps if absolute else switch_eps * v0norm
    return np.array([tau * 1e-3, tau * 1e-2, tau * 1e-1, tau], np.float64)


def cg_solve(D: DistMatrix, b_local, tol=1e-10, max_iter=1000, mode="dynamic", switch_eps=None) -> DistResult:
    """Distributed CG (Alg. 1) from x0 = 0; b_local: this rank's slice of b (engine vector)."""
    E, C = D.engine, D.comm
    dev = D.comm_device
    nl = D.row_end - D.row_begin
    off = D.row_begin - D.xlo
    xe = E.vector(D.xhi - D.xlo)
    p = xe[off:off + nl]
    r = E.vector(nl)
    r.copy_(b_local)
    x = E.vector(nl)
    mu = E.vector(nl)
    bb, rr = C.allsum([E.dot(D.M, b_local, b_local), E.dot(D.M, r, r)], dev)
    nb, rho = math.sqrt(bb), rr
    hist = []
    if nb == 0.0:
        return DistResult(x, 0, True, 0.0, np.zeros(1), row_begin=D.row_begin, row_end=D.row_end)
    p.copy_(r)
    eps = tol if switch_eps is None else switch_eps
    th = thresholds(eps, math.sqrt(rho), D.n) if mode == "dynamic" else None
    converged, status, j = False, "ok", 0
    while True:
        relres = math.sqrt(rho) / nb
        hist.append(relres)
        if relres < tol:
            converged = True
            break
        if j == max_iter:
            break
        C.halo(xe, D.xlo, D.plan)
        level = E.levels(xe, th) if th is not None else None
        E.spmv(D.M, xe, mu, level)
        sigma, = C.allsum([E.dot(D.M, mu, p)], dev)
        if not (sigma > 0.0) or not math.isfinite(sigma):
            status = "breakdown"
            break
        alpha = rho / sigma
        rr, = C.allsum([E.update_xr(D.M, alpha, p, mu, x, r)], dev)
        beta = rr / rho
        rho = rr
        E.update_p(D.M, beta, r, p)
        j += 1
    return DistResult(x, j, converged, hist[-1], np.array(hist), status, D.plan.bytes_per_exchange() * j,
                      D.row_begin, D.row_end)
