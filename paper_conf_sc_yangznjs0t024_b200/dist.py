"""Row-block multi-GPU solves through libmf's C ABI (include/mf.h).

The paper's solver is single-GPU.  For matrices too large for one GPU (C5) the rows are
split into contiguous blocks of whole 16-row tile rows, one block per GPU, one process per GPU.
Everything runs inside libmf: the halo plan, the NCCL halo exchange of the SpMV input, the staged
tile SpMV, the deterministic rank-ordered reductions, every scalar of the iteration (device
side) and the stop test (device flag).  This module only marshals arguments: it partitions the
rows, ships NCCL's 128-byte unique id from rank 0 to the other ranks with torch.distributed,
and wraps the handles.  With one rank a solve is bit-identical to mf_cg_solve / mf_bicgstab_solve.
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass

import numpy as np

TS = 16


# ------------------------------------------------------------------ partition (host)
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


def local_rows(A, row_begin: int, row_end: int):
    """Rows [row_begin, row_end) of a host CSR (global column ids): (rowptr, colidx, vals)."""
    a, b = int(A.rowptr[row_begin]), int(A.rowptr[row_end])
    return (np.ascontiguousarray(A.rowptr[row_begin:row_end + 1] - a), np.ascontiguousarray(A.colidx[a:b]),
            np.ascontiguousarray(A.vals[a:b]))


def halo_plan(n_global: int, rank_rows, rank: int, colidx):
    """libmf's host planner (mf_dist_plan): (halo segments ascending, recv counts per rank)."""
    from . import _check, lib
    rr = np.ascontiguousarray(rank_rows, np.int64)
    ci = np.ascontiguousarray(colidx, np.int32)
    P = len(rr) - 1
    counts = np.zeros(P, np.int64)
    nh = C.c_int64()
    _check(lib().mf_dist_plan(int(n_global), P, C.c_void_p(rr.ctypes.data), int(rank), ci.size,
                              C.c_void_p(ci.ctypes.data), C.c_void_p(counts.ctypes.data), None, 0, C.byref(nh)))
    segs = np.zeros(max(nh.value, 1), np.int32)
    _check(lib().mf_dist_plan(int(n_global), P, C.c_void_p(rr.ctypes.data), int(rank), ci.size,
                              C.c_void_p(ci.ctypes.data), C.c_void_p(counts.ctypes.data), C.c_void_p(segs.ctypes.data),
                              segs.size, C.byref(nh)))
    return segs[:nh.value], counts


# ------------------------------------------------------------------ communicator
class Comm:
    """An mf_comm over the processes of a torch.distributed group (one GPU each): rank 0 makes
    NCCL's unique id, torch.distributed broadcasts its 128 bytes, libmf creates the NCCL comm."""

    def __init__(self, group=None):
        import torch
        import torch.distributed as td

        from . import _check, lib
        self.size = td.get_world_size(group)
        self.rank = td.get_rank(group)
        uid = np.zeros(128, np.uint8)
        if self.rank == 0:
            _check(lib().mf_nccl_unique_id(C.c_void_p(uid.ctypes.data)))
        dev = torch.device("cuda", torch.cuda.current_device()) if td.get_backend(group) == "nccl" else "cpu"
        t = torch.from_numpy(uid).to(dev)
        src = 0 if group is None else td.get_global_rank(group, 0)
        td.broadcast(t, src=src, group=group)
        uid = np.ascontiguousarray(t.cpu().numpy())
        h = C.c_void_p()
        _check(lib().mf_comm_create(C.c_void_p(uid.ctypes.data), self.size, self.rank, C.byref(h)))
        self._h = h

    def close(self):
        if getattr(self, "_h", None):
            from . import lib
            lib().mf_comm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class LocalGroup:
    """In-process rank group (mf_local_group): `nranks` host threads of this process each drive one
    rank, all on the current GPU.  Only the device-initiated kernel (dist_mode 2) runs on it; it
    checks the multi-rank exchange where one GPU is all there is.  Each rank's thread must use its
    own CUDA stream (torch.cuda.stream), and the ranks' plans must fit the GPU together
    (grid_ctas <= SMs / nranks)."""

    def __init__(self, nranks: int):
        from . import _check, lib
        h = C.c_void_p()
        _check(lib().mf_local_group_create(int(nranks), C.byref(h)))
        self._h = h
        self.size = int(nranks)

    def comm(self, rank: int) -> "LocalComm":
        return LocalComm(self, rank)

    def close(self):
        if getattr(self, "_h", None):
            from . import lib
            lib().mf_local_group_destroy(self._h)
            self._h = None


class LocalComm(Comm):
    """Rank `rank` of a LocalGroup (an mf_comm without NCCL)."""

    def __init__(self, group: LocalGroup, rank: int):   # noqa: super().__init__ is the NCCL path
        from . import _check, lib
        h = C.c_void_p()
        _check(lib().mf_comm_create_local(group._h, int(rank), C.byref(h)))
        self._h = h
        self.size, self.rank, self.group = group.size, int(rank), group


class DistTileMatrix:
    """This rank's rows [row_begin, row_end) of an n_global x n_global matrix
    (mf_tile_matrix_from_csr_dist): device CSR with local rowptr and GLOBAL column ids."""

    def __init__(self, comm: Comm, n_global, row_begin, row_end, rowptr, colidx, vals, classify=True, grid_ctas=0,
                 block_threads=0, layout=0, stream=None):
        import torch

        from . import ConvertOpts, _check, _need_cuda, _ptr, _stream_ptr, lib
        _need_cuda(rowptr, torch.int64, "rowptr")
        _need_cuda(colidx, torch.int32, "colidx")
        _need_cuda(vals, torch.float64, "vals")
        o = ConvertOpts(int(bool(classify)), 1e-15, int(grid_ctas), int(block_threads), int(layout))
        h = C.c_void_p()
        self._h = None
        _check(lib().mf_tile_matrix_from_csr_dist(comm._h, int(n_global), int(row_begin), int(row_end), int(colidx.numel()),
                                                  _ptr(rowptr), _ptr(colidx), _ptr(vals), C.byref(o), _stream_ptr(stream),
                                                  C.byref(h)))
        self._h = h
        self.comm = comm
        self.n_global, self.row_begin, self.row_end = int(n_global), int(row_begin), int(row_end)
        self.n_rows = self.n_cols = self.row_end - self.row_begin

    @classmethod
    def from_host_csr(cls, comm: Comm, A, row_begin, row_end, device="cuda", **kw):
        import torch
        rp, ci, va = local_rows(A, row_begin, row_end)
        t = lambda a: torch.from_numpy(a).to(device)   # noqa: E731
        return cls(comm, A.n_rows, row_begin, row_end, t(rp), t(ci), t(va), **kw)

    def dist_info(self) -> dict:
        from . import _check, lib
        v = [C.c_int64() for _ in range(4)]
        _check(lib().mf_dist_info(self._h, *[C.byref(x) for x in v]))
        return dict(zip(("row_begin", "row_end", "halo_segments", "send_segments"), (x.value for x in v)))

    def info(self) -> dict:
        from . import TileMatrix
        return TileMatrix.info(self)

    def export(self, stream=None) -> dict:
        from . import TileMatrix
        return TileMatrix.export(self, stream)

    def plan(self):
        from . import TileMatrix
        return TileMatrix.plan(self)

    def close(self):
        if getattr(self, "_h", None):
            from . import lib
            lib().mf_tile_matrix_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _solve_dist(fn_name, A: DistTileMatrix, b_local, **kw):
    from . import _solve, lib
    return _solve(getattr(lib(), fn_name), A, b_local, **kw)


def cg_solve(A: DistTileMatrix, b_local, **kw):
    """Distributed CG (Alg. 1) over the communicator: b_local, the result x are this rank's slices."""
    return _solve_dist("mf_cg_solve_dist", A, b_local, **kw)


def bicgstab_solve(A: DistTileMatrix, b_local, **kw):
    """Distributed BiCGSTAB (Alg. 2)."""
    return _solve_dist("mf_bicgstab_solve_dist", A, b_local, **kw)


@dataclass
class Partition:
    bounds: list
    rank: int

    @property
    def rows(self):
        return self.bounds[self.rank], self.bounds[self.rank + 1]
