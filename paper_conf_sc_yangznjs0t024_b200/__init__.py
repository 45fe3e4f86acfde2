"""Python binding of libmf (include/mf.h): the B200-native Mille-feuille hot path.

Argument marshalling only: every step of the method (conversion, SpMV, levels, dots, the
persistent CG / BiCGSTAB kernels, ILU(0) apply) runs in the CUDA kernels of
``csrc/``.  PyTorch provides device memory (the library allocates through torch's caching
allocator), streams and process groups.  There is no CPU fallback: without ``libmf.so`` or
without a B200 every call raises ``MFError``.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading
from dataclasses import dataclass

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB_PATH = os.path.join(HERE, "libmf.so")
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(ROOT, "include")

FP64, FP32, FP16, FP8, BYPASS = 0, 1, 2, 3, 4
MODE_FP64, MODE_STATIC, MODE_DYNAMIC = 0, 1, 2

STATUS = {0: "MF_OK", 1: "MF_ERR_INVALID_ARG", 2: "MF_ERR_UNSORTED_CSR", 3: "MF_ERR_NONFINITE", 4: "MF_ERR_OOM",
          5: "MF_ERR_CUDA", 6: "MF_ERR_NCCL", 7: "MF_ERR_BREAKDOWN", 8: "MF_ERR_ZERO_PIVOT", 9: "MF_ERR_DEADLOCK",
          10: "MF_ERR_UNSUPPORTED_DEVICE", 11: "MF_ERR_NOT_IMPLEMENTED", 12: "MF_ERR_UNSUPPORTED"}

# every symbol include/mf.h declares
SYMBOLS = ["mf_default_convert_opts", "mf_default_solve_opts", "mf_set_allocator", "mf_tile_matrix_from_csr",
           "mf_tile_matrix_destroy", "mf_tile_matrix_info", "mf_tile_matrix_export", "mf_spmv", "mf_levels",
           "mf_dot", "mf_precond_create", "mf_precond_create_ex", "mf_precond_info", "mf_precond_destroy",
           "mf_precond_apply", "mf_cg_solve",
           "mf_bicgstab_solve", "mf_cg_update_xr", "mf_cg_update_p", "mf_status_string", "mf_last_error",
           "mf_abi_version", "mf_nccl_unique_id", "mf_comm_create", "mf_comm_destroy", "mf_comm_info",
           "mf_tile_matrix_from_csr_dist", "mf_cg_solve_dist", "mf_bicgstab_solve_dist", "mf_dist_info", "mf_dist_plan",
           "mf_local_group_create", "mf_local_group_destroy", "mf_comm_create_local"]

NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17", "-fmad=false",
              "-Xcompiler", "-fPIC"]


class MFError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        super().__init__(f"{STATUS.get(status, status)}: {detail}")


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile libmf.so in-tree for sm_100a (nvcc cross-compiles without a GPU)."""
    srcs = sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".cu"))
    deps = srcs + [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".cuh")] + \
        [os.path.join(INCLUDE, "mf.h")]
    if not force and os.path.exists(LIB_PATH) and \
            os.path.getmtime(LIB_PATH) >= max(os.path.getmtime(d) for d in deps):
        return LIB_PATH
    nccl_inc, nccl_lib = _nccl_paths()
    # one nvcc per translation unit, in parallel (no relocatable device code: each kernel's
    # device code lives in the object of its host stub), then one shared-library link
    from concurrent.futures import ThreadPoolExecutor
    objdir = os.path.join(HERE, "build")
    os.makedirs(objdir, exist_ok=True)
    objs = [os.path.join(objdir, os.path.basename(s)[:-3] + ".o") for s in srcs]
    cmds = [["nvcc", *NVCC_FLAGS, "-I", INCLUDE, "-I", nccl_inc, "-c", "-o", o, s] for s, o in zip(srcs, objs)]
    if verbose:
        for c in cmds:
            print(" ".join(c))
    with ThreadPoolExecutor(len(cmds)) as ex:
        for f in [ex.submit(subprocess.check_call, c) for c in cmds]:
            f.result()
    tmp = LIB_PATH + f".{os.getpid()}.tmp"
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, *objs,
                           "-L", nccl_lib, "-l:libnccl.so.2", f"-Xlinker=-rpath={nccl_lib}"])
    os.replace(tmp, LIB_PATH)
    return LIB_PATH


def _nccl_paths():
    import nvidia.nccl as nn
    base = os.path.dirname(nn.__file__) if getattr(nn, "__file__", None) else list(nn.__path__)[0]
    return os.path.join(base, "include"), os.path.join(base, "lib")


# ------------------------------------------------------------------ ctypes structs (mirror mf.h)
class ConvertOpts(C.Structure):
    _fields_ = [("classify", C.c_int32), ("loss_tol", C.c_double), ("grid_ctas", C.c_int32),
                ("block_threads", C.c_int32), ("layout", C.c_int32)]


class TileInfo(C.Structure):
    _fields_ = [("n_rows", C.c_int64), ("n_cols", C.c_int64), ("nnz", C.c_int64), ("T", C.c_int32),
                ("tilenum", C.c_int64), ("rownum", C.c_int64), ("n_tile_rows", C.c_int64),
                ("tiles_per_prec", C.c_int64 * 4), ("nval", C.c_int64 * 4), ("max_tiles_per_tile_row", C.c_int64),
                ("slots", C.c_int64), ("canonical_bytes", C.c_int64), ("csr_bytes", C.c_int64),
                ("kernel_bytes", C.c_int64), ("plan_G", C.c_int32), ("plan_B", C.c_int32), ("convert_ms", C.c_double),
                ("convert_launches", C.c_int64), ("layout", C.c_int32)]


class TileExport(C.Structure):
    _fields_ = [(n, C.c_void_p) for n in ("TileRowidx", "TileColidx", "TilePrec", "Floor", "TileNnz", "Nonrow",
                                           "ValOff", "TileRowPtr", "RowIndex", "CsrRowptr", "CsrColidx", "Val64",
                                           "Val32", "Val16", "Val8", "PlanRows")]


class SolveOpts(C.Structure):
    _fields_ = [("tol", C.c_double), ("max_iter", C.c_int64), ("mode", C.c_int32), ("switch_eps", C.c_double),
                ("switch_absolute", C.c_int32), ("sticky", C.c_int32), ("range_guard", C.c_int32),
                ("M", C.c_void_p), ("residual_history", C.c_void_p), ("history_cap", C.c_int64),
                ("tile_level_counts", C.c_void_p), ("level_counts_cap", C.c_int64), ("collect_stats", C.c_int32),
                ("watchdog_ms", C.c_int32), ("cg_variant", C.c_int32), ("dist_mode", C.c_int32)]


class SolveInfo(C.Structure):
    _fields_ = [("iterations", C.c_int64), ("converged", C.c_int32), ("status", C.c_int32),
                ("rel_residual", C.c_double), ("kernel_ms", C.c_double), ("model_bytes", C.c_double),
                ("n_spmv", C.c_int64), ("launches", C.c_int64), ("barrier_ms", C.c_double),
                ("phase_ms", C.c_double * 12), ("ring_slots", C.c_int32), ("mu_onchip", C.c_int32)]


_lib = None
_lock = threading.Lock()
_ALLOC_CB = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
_FREE_CB = C.CFUNCTYPE(None, C.c_void_p, C.c_void_p, C.c_void_p)
_callbacks = []


def lib():
    """Load libmf.so (built in-tree).  Raises MFError if it is missing: there is no fallback."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        if not os.path.exists(LIB_PATH):
            raise MFError(5, f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback)")
        L = C.CDLL(LIB_PATH)
        vp, i64, i32, d = C.c_void_p, C.c_int64, C.c_int32, C.c_double
        L.mf_status_string.restype = C.c_char_p
        L.mf_status_string.argtypes = [C.c_int]
        L.mf_last_error.restype = C.c_char_p
        L.mf_abi_version.restype = C.c_int32
        L.mf_default_convert_opts.argtypes = [C.POINTER(ConvertOpts)]
        L.mf_default_solve_opts.argtypes = [C.POINTER(SolveOpts)]
        L.mf_set_allocator.argtypes = [_ALLOC_CB, _FREE_CB, vp]
        L.mf_tile_matrix_from_csr.argtypes = [i64, i64, i64, vp, vp, vp, C.POINTER(ConvertOpts), vp, C.POINTER(vp)]
        L.mf_tile_matrix_destroy.argtypes = [vp]
        L.mf_tile_matrix_info.argtypes = [vp, C.POINTER(TileInfo)]
        L.mf_tile_matrix_export.argtypes = [vp, C.POINTER(TileExport), vp]
        L.mf_spmv.argtypes = [vp, vp, vp, vp, i32, vp, vp]
        L.mf_levels.argtypes = [vp, i64, vp, vp, vp]
        L.mf_dot.argtypes = [vp, vp, vp, C.POINTER(d), vp]
        L.mf_precond_create.argtypes = [vp, C.c_int, vp, C.POINTER(vp)]
        L.mf_precond_create_ex.argtypes = [vp, C.POINTER(PrecondOpts), vp, C.POINTER(vp)]
        L.mf_precond_info.argtypes = [vp, C.POINTER(PrecondStats)]
        L.mf_precond_destroy.argtypes = [vp]
        L.mf_precond_apply.argtypes = [vp, vp, vp, vp]
        L.mf_cg_solve.argtypes = [vp, vp, vp, C.POINTER(SolveOpts), C.POINTER(SolveInfo), vp]
        L.mf_bicgstab_solve.argtypes = [vp, vp, vp, C.POINTER(SolveOpts), C.POINTER(SolveInfo), vp]
        L.mf_cg_update_xr.argtypes = [vp, d, vp, vp, vp, vp, C.POINTER(d), vp]
        L.mf_cg_update_p.argtypes = [vp, d, vp, vp, vp]
        L.mf_nccl_unique_id.argtypes = [vp]
        L.mf_comm_create.argtypes = [vp, i32, i32, C.POINTER(vp)]
        L.mf_comm_destroy.argtypes = [vp]
        L.mf_comm_info.argtypes = [vp, C.POINTER(i32), C.POINTER(i32)]
        L.mf_tile_matrix_from_csr_dist.argtypes = [vp, i64, i64, i64, i64, vp, vp, vp, C.POINTER(ConvertOpts), vp,
                                                   C.POINTER(vp)]
        L.mf_cg_solve_dist.argtypes = [vp, vp, vp, C.POINTER(SolveOpts), C.POINTER(SolveInfo), vp]
        L.mf_bicgstab_solve_dist.argtypes = [vp, vp, vp, C.POINTER(SolveOpts), C.POINTER(SolveInfo), vp]
        L.mf_dist_info.argtypes = [vp, C.POINTER(i64), C.POINTER(i64), C.POINTER(i64), C.POINTER(i64)]
        L.mf_dist_plan.argtypes = [i64, i32, vp, i32, i64, vp, vp, vp, i64, C.POINTER(i64)]
        L.mf_local_group_create.argtypes = [i32, C.POINTER(vp)]
        L.mf_local_group_destroy.argtypes = [vp]
        L.mf_comm_create_local.argtypes = [vp, i32, C.POINTER(vp)]
        _lib = L
        return L


def _check(status: int):
    if status != 0:
        raise MFError(status, lib().mf_last_error().decode())


def use_torch_allocator():
    """Route libmf's device allocations through torch's caching allocator."""
    import torch

    def _alloc(size, stream, ctx):
        try:
            return torch.cuda.caching_allocator_alloc(int(size), torch.cuda.current_device(), stream or 0)
        except Exception:
            return None

    def _free(ptr, stream, ctx):
        torch.cuda.caching_allocator_delete(ptr)

    cb = (_ALLOC_CB(_alloc), _FREE_CB(_free))
    _callbacks.append(cb)
    _check(lib().mf_set_allocator(cb[0], cb[1], None))


def _stream_ptr(stream=None):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def _ptr(t):
    return C.c_void_p(t.data_ptr()) if t is not None else None


def _need_cuda(t, dtype, name):
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda or t.dtype != dtype or not t.is_contiguous():
        raise MFError(1, f"{name} must be a contiguous CUDA {dtype} tensor")


# ------------------------------------------------------------------ the tile matrix
class TileMatrix:
    """Handle to an mf_tile_matrix (device CSR -> two-level tiles)."""

    def __init__(self, n_rows, n_cols, rowptr, colidx, vals, classify=True, loss_tol=1e-15, grid_ctas=0,
                 block_threads=0, layout=0, stream=None):
        import torch
        _need_cuda(rowptr, torch.int64, "rowptr")
        _need_cuda(colidx, torch.int32, "colidx")
        _need_cuda(vals, torch.float64, "vals")
        L = lib()
        o = ConvertOpts(int(bool(classify)), float(loss_tol), int(grid_ctas), int(block_threads), int(layout))
        h = C.c_void_p()
        self._h = None
        _check(L.mf_tile_matrix_from_csr(int(n_rows), int(n_cols), int(colidx.numel()), _ptr(rowptr), _ptr(colidx),
                                         _ptr(vals), C.byref(o), _stream_ptr(stream), C.byref(h)))
        self._h = h
        self.n_rows, self.n_cols = int(n_rows), int(n_cols)

    @classmethod
    def from_host_csr(cls, A, device="cuda", **kw):
        """Copy a host CSR (workloads.CSR-like: n_rows, n_cols, rowptr, colidx, vals) and convert."""
        import torch
        rp = torch.from_numpy(np.ascontiguousarray(A.rowptr, np.int64)).to(device)
        ci = torch.from_numpy(np.ascontiguousarray(A.colidx, np.int32)).to(device)
        va = torch.from_numpy(np.ascontiguousarray(A.vals, np.float64)).to(device)
        return cls(A.n_rows, A.n_cols, rp, ci, va, **kw)

    def close(self):
        if getattr(self, "_h", None):
            lib().mf_tile_matrix_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def info(self) -> dict:
        inf = TileInfo()
        _check(lib().mf_tile_matrix_info(self._h, C.byref(inf)))
        out = {f: getattr(inf, f) for f, _ in TileInfo._fields_}
        out["tiles_per_prec"] = list(inf.tiles_per_prec)
        out["nval"] = list(inf.nval)
        return out

    def export(self, stream=None) -> dict:
        """The canonical arrays (bit-exact contract) plus PlanRows, as numpy."""
        inf = self.info()
        nt, nr, nz = inf["tilenum"], inf["rownum"], inf["nnz"]
        arrs = {"TileRowidx": np.empty(nt, np.int32), "TileColidx": np.empty(nt, np.int32),
                "TilePrec": np.empty(nt, np.uint8), "Floor": np.empty(nt, np.uint8),
                "TileNnz": np.empty(nt + 1, np.int64), "Nonrow": np.empty(nt + 1, np.int64),
                "ValOff": np.empty(nt, np.int64), "TileRowPtr": np.empty(inf["n_tile_rows"] + 1, np.int64),
                "RowIndex": np.empty(nr, np.uint8), "CsrRowptr": np.empty(nr, np.uint8),
                "CsrColidx": np.empty(nz, np.uint8), "Val64": np.empty(inf["nval"][0], np.float64),
                "Val32": np.empty(inf["nval"][1], np.float32), "Val16": np.empty(inf["nval"][2], np.uint16),
                "Val8": np.empty(inf["nval"][3], np.uint8), "PlanRows": np.empty(inf["plan_G"] + 1, np.int64)}
        ex = TileExport(**{k: v.ctypes.data for k, v in arrs.items()})
        _check(lib().mf_tile_matrix_export(self._h, C.byref(ex), _stream_ptr(stream)))
        return arrs

    def plan(self):
        inf = self.info()
        return inf["plan_G"], inf["plan_B"], self.export()["PlanRows"]

    def spmv(self, x, level=None, range_guard=True, counts=False, out=None, stream=None):
        import torch
        _need_cuda(x, torch.float64, "x")
        y = out if out is not None else torch.empty(self.n_rows, dtype=torch.float64, device=x.device)
        if level is not None:
            _need_cuda(level, torch.uint8, "level")
        c = np.zeros(5, np.int64) if counts else None
        _check(lib().mf_spmv(self._h, _ptr(x), _ptr(y), _ptr(level), int(bool(range_guard)),
                             C.c_void_p(c.ctypes.data) if c is not None else None, _stream_ptr(stream)))
        return (y, c) if counts else y

    def dot(self, u, v, stream=None) -> float:
        import torch
        _need_cuda(u, torch.float64, "u")
        _need_cuda(v, torch.float64, "v")
        out = C.c_double()
        _check(lib().mf_dot(self._h, _ptr(u), _ptr(v), C.byref(out), _stream_ptr(stream)))
        return out.value


    # CG steps C and D (Alg. 1) on this matrix's rows -- the per-rank kernels of the
    # row-block multi-GPU driver (dist.py); same reduction tree as dot().
    def cg_update_xr(self, alpha, p, mu, x, r, stream=None) -> float:
        """x += alpha p ; r = fma(-alpha, mu, r) ; returns (r, r)."""
        import torch
        for t, nm in ((p, "p"), (mu, "mu"), (x, "x"), (r, "r")):
            _need_cuda(t, torch.float64, nm)
        out = C.c_double()
        _check(lib().mf_cg_update_xr(self._h, float(alpha), _ptr(p), _ptr(mu), _ptr(x), _ptr(r), C.byref(out),
                                     _stream_ptr(stream)))
        return out.value

    def cg_update_p(self, beta, r, p, stream=None):
        """p = fma(beta, p, r)."""
        import torch
        _need_cuda(r, torch.float64, "r")
        _need_cuda(p, torch.float64, "p")
        _check(lib().mf_cg_update_p(self._h, float(beta), _ptr(r), _ptr(p), _stream_ptr(stream)))


def levels(v, th, stream=None):
    """Alg. 4: level of every 16-element segment of v (device) for thresholds th (4 floats)."""
    import torch
    _need_cuda(v, torch.float64, "v")
    out = torch.empty((v.numel() + 15) // 16, dtype=torch.uint8, device=v.device)
    th = np.ascontiguousarray(th, np.float64)
    _check(lib().mf_levels(_ptr(v), v.numel(), C.c_void_p(th.ctypes.data), _ptr(out), _stream_ptr(stream)))
    return out


@dataclass
class SolveResult:
    x: object
    iterations: int
    converged: bool
    status: int
    rel_residual: float
    kernel_ms: float
    model_bytes: float
    n_spmv: int
    launches: int
    barrier_ms: float
    phase_ms: list
    history: np.ndarray | None
    level_counts: np.ndarray | None


def _solve(fn, A: TileMatrix, b, x0=None, tol=1e-10, max_iter=1000, mode=MODE_DYNAMIC, switch_eps=None,
           switch_absolute=False, range_guard=True, sticky=False, history=True, level_counts=False,
           collect_stats=False, M=None, stream=None, raise_on_breakdown=True, watchdog_ms=0,
           cg_variant=0, dist_mode=0) -> SolveResult:
    import torch
    _need_cuda(b, torch.float64, "b")
    x = torch.zeros_like(b) if x0 is None else x0.clone()
    hist = np.full(max_iter + 2, np.nan) if history else None
    lc = np.zeros((2 * max_iter + 2, 5), np.int64) if level_counts else None
    o = SolveOpts()
    lib().mf_default_solve_opts(C.byref(o))
    o.tol, o.max_iter, o.mode = float(tol), int(max_iter), int(mode)
    o.switch_eps = -1.0 if switch_eps is None else float(switch_eps)
    o.switch_absolute, o.range_guard, o.sticky = int(switch_absolute), int(range_guard), int(sticky)
    o.M = M._h if M is not None else None
    if hist is not None:
        o.residual_history, o.history_cap = hist.ctypes.data, hist.size
    if lc is not None:
        o.tile_level_counts, o.level_counts_cap = lc.ctypes.data, lc.shape[0]
    o.collect_stats = int(collect_stats)
    o.watchdog_ms = int(watchdog_ms)
    o.cg_variant = int(cg_variant)
    o.dist_mode = int(dist_mode)
    info = SolveInfo()
    st = fn(A._h, _ptr(b), _ptr(x), C.byref(o), C.byref(info), _stream_ptr(stream))
    if st != 0 and (raise_on_breakdown or st != 7):
        raise MFError(st, lib().mf_last_error().decode())
    k = info.iterations
    return SolveResult(x, k, bool(info.converged), info.status, info.rel_residual, info.kernel_ms,
                       info.model_bytes, info.n_spmv, info.launches, info.barrier_ms, list(info.phase_ms),
                       hist[: k + 1] if hist is not None else None,
                       lc[: info.n_spmv] if lc is not None else None)


def cg_solve(A: TileMatrix, b, **kw) -> SolveResult:
    """Single-kernel (P)CG (Alg. 1 / Alg. 3)."""
    return _solve(lib().mf_cg_solve, A, b, **kw)


def bicgstab_solve(A: TileMatrix, b, **kw) -> SolveResult:
    """Single-kernel (P)BiCGSTAB (Alg. 2)."""
    return _solve(lib().mf_bicgstab_solve, A, b, **kw)


SPTRSV_SYNC_FREE, SPTRSV_RECURSIVE_BLOCK = 0, 1


class PrecondOpts(C.Structure):
    _fields_ = [("kind", C.c_int), ("sptrsv", C.c_int32), ("rb_depth", C.c_int32)]


class PrecondStats(C.Structure):
    _fields_ = [("rb_depth", C.c_int32), ("nodes_l", C.c_int32), ("nodes_u", C.c_int32), ("sweep", C.c_int32),
                ("depth_l", C.c_int64), ("depth_u", C.c_int64), ("nnz_l", C.c_int64), ("nnz_u", C.c_int64)]


class Precond:
    """ILU(0) of the stored matrix; z = M^-1 r by SpTRSV kernels.  sptrsv =
    SPTRSV_RECURSIVE_BLOCK selects the recursive block SpTRSV of P:166 (rb_depth levels, 0 = auto)."""

    def __init__(self, A: TileMatrix, kind: int = 1, stream=None, sptrsv: int = SPTRSV_SYNC_FREE, rb_depth: int = 0):
        h = C.c_void_p()
        self._h = None
        o = PrecondOpts(int(kind), int(sptrsv), int(rb_depth))
        _check(lib().mf_precond_create_ex(A._h, C.byref(o), _stream_ptr(stream), C.byref(h)))
        self._h = h
        self.n = A.n_rows

    def info(self) -> dict:
        st = PrecondStats()
        _check(lib().mf_precond_info(self._h, C.byref(st)))
        return {f: getattr(st, f) for f, _ in PrecondStats._fields_}

    def apply(self, r, out=None, stream=None):
        import torch
        _need_cuda(r, torch.float64, "r")
        z = out if out is not None else torch.empty_like(r)
        _check(lib().mf_precond_apply(self._h, _ptr(r), _ptr(z), _stream_ptr(stream)))
        return z

    def close(self):
        if getattr(self, "_h", None):
            lib().mf_precond_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
