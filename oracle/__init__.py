"""ctypes wrapper around oracle/mf_oracle.c -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this module.  It never imports the CUDA package
``paper_conf_sc_yangznjs0t024_b200`` and the CUDA package never imports it.

Every function here only marshals numpy arrays into the C oracle; the arithmetic lives in
``mf_oracle.c`` (see its header for the PAPER.md citations and the pins).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mf_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

# precision codes (PAPER.md P:212 encodes differently; this build uses SURVEY 8b's order)
FP64, FP32, FP16, FP8, BYPASS = 0, 1, 2, 3, 4
MODE_FP64, MODE_STATIC, MODE_DYNAMIC = 0, 1, 2
OK, ERR_INVALID_ARG, ERR_UNSORTED_CSR, ERR_NONFINITE, ERR_OOM = 0, 1, 2, 3, 4
ERR_BREAKDOWN, ERR_ZERO_PIVOT = 7, 8


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C11, no FMA contraction)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".{os.getpid()}.tmp"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-ffp-contract=off", "-fopenmp",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


class _Tiles(C.Structure):
    _fields_ = [("n_rows", C.c_int64), ("n_cols", C.c_int64), ("nnz", C.c_int64), ("T", C.c_int32),
                ("tilenum", C.c_int64), ("rownum", C.c_int64), ("n_tile_rows", C.c_int64),
                ("TileRowidx", C.POINTER(C.c_int32)), ("TileColidx", C.POINTER(C.c_int32)),
                ("TilePrec", C.POINTER(C.c_uint8)), ("Floor", C.POINTER(C.c_uint8)),
                ("TileNnz", C.POINTER(C.c_int64)), ("Nonrow", C.POINTER(C.c_int64)),
                ("ValOff", C.POINTER(C.c_int64)), ("TileRowPtr", C.POINTER(C.c_int64)),
                ("RowIndex", C.POINTER(C.c_uint8)), ("CsrRowptr", C.POINTER(C.c_uint8)),
                ("CsrColidx", C.POINTER(C.c_uint8)),
                ("Val64", C.POINTER(C.c_double)), ("Val32", C.POINTER(C.c_float)),
                ("Val16", C.POINTER(C.c_uint16)), ("Val8", C.POINTER(C.c_uint8)),
                ("nval", C.c_int64 * 4)]


class _Plan(C.Structure):
    _fields_ = [("G", C.c_int32), ("B", C.c_int32), ("R", C.POINTER(C.c_int64)), ("P", C.c_int32),
                ("Gr", C.POINTER(C.c_int32))]


class _Opts(C.Structure):
    _fields_ = [("tol", C.c_double), ("max_iter", C.c_int64), ("mode", C.c_int32),
                ("switch_eps", C.c_double), ("switch_absolute", C.c_int32), ("sticky", C.c_int32),
                ("range_guard", C.c_int32)]


class _Info(C.Structure):
    _fields_ = [("iterations", C.c_int64), ("converged", C.c_int32), ("status", C.c_int32),
                ("rel_residual", C.c_double), ("n_spmv", C.c_int64)]


class _Sticky(C.Structure):
    _fields_ = [("cur", C.POINTER(C.c_uint8)), ("wv", C.POINTER(C.c_double))]


class _Ilu(C.Structure):
    _fields_ = [("n", C.c_int64), ("rowptr", C.POINTER(C.c_int64)), ("colidx", C.POINTER(C.c_int32)),
                ("lu", C.POINTER(C.c_double)), ("diag", C.POINTER(C.c_int64)), ("rb_depth", C.c_int32)]


def _p(a, ctype):
    return a.ctypes.data_as(C.POINTER(ctype)) if a is not None else None


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = C.CDLL(build())
            d, i64, i32, u8, vp = C.c_double, C.c_int64, C.c_int32, C.c_uint8, C.c_void_p
            L.orc_rne.argtypes = [d, C.c_int]; L.orc_rne.restype = d
            L.orc_classify.argtypes = [d, d]; L.orc_classify.restype = C.c_int
            L.orc_fp16_bits.argtypes = [d]; L.orc_fp16_bits.restype = C.c_uint16
            L.orc_fp16_value.argtypes = [C.c_uint16]; L.orc_fp16_value.restype = d
            L.orc_e4m3_bits.argtypes = [d]; L.orc_e4m3_bits.restype = u8
            L.orc_e4m3_value.argtypes = [u8]; L.orc_e4m3_value.restype = d
            L.orc_tiles_build.argtypes = [i64, i64, i64, vp, vp, vp, i32, C.c_int, d, C.POINTER(_Tiles)]
            L.orc_tiles_build.restype = C.c_int
            L.orc_tiles_free.argtypes = [C.POINTER(_Tiles)]; L.orc_tiles_free.restype = None
            L.orc_tile_value.argtypes = [C.POINTER(_Tiles), i64, i64]; L.orc_tile_value.restype = d
            L.orc_tiles_stored_csr.argtypes = [C.POINTER(_Tiles), vp, vp, vp]
            L.orc_tiles_stored_csr.restype = None
            L.orc_levels.argtypes = [vp, i64, i32, vp, vp]; L.orc_levels.restype = None
            L.orc_tile_eff.argtypes = [C.POINTER(_Tiles), vp, C.c_int, vp]; L.orc_tile_eff.restype = None
            L.orc_spmv_tiles.argtypes = [C.POINTER(_Tiles), vp, vp, vp, C.c_int, vp, vp]
            L.orc_spmv_tiles.restype = None
            L.orc_spmv_csr.argtypes = [i64, vp, vp, vp, vp, vp]; L.orc_spmv_csr.restype = None
            L.orc_dot.argtypes = [vp, vp, i64, C.POINTER(_Plan)]; L.orc_dot.restype = d
            solver_args = [C.POINTER(_Tiles), C.POINTER(_Ilu), vp, vp, C.POINTER(_Opts), C.POINTER(_Plan),
                           vp, i64, vp, i64, C.POINTER(_Info)]
            L.orc_pcg.argtypes = solver_args; L.orc_pcg.restype = C.c_int
            L.orc_pbicgstab.argtypes = solver_args; L.orc_pbicgstab.restype = C.c_int
            L.orc_cg_single_reduction.argtypes = [C.POINTER(_Tiles), vp, vp, C.POINTER(_Opts), C.POINTER(_Plan),
                                                  vp, i64, vp, i64, C.POINTER(_Info)]
            L.orc_cg_single_reduction.restype = C.c_int
            L.orc_cg_csr.argtypes = [i64, vp, vp, vp, vp, vp, d, i64, vp, i64, C.POINTER(_Info)]
            L.orc_cg_csr.restype = C.c_int
            L.orc_true_relres.argtypes = [i64, vp, vp, vp, vp, vp]; L.orc_true_relres.restype = d
            L.orc_ilu0.argtypes = [i64, vp, vp, vp, vp, vp]; L.orc_ilu0.restype = C.c_int
            L.orc_ilu_apply.argtypes = [C.POINTER(_Ilu), vp, vp]; L.orc_ilu_apply.restype = None
            L.orc_csr_validate.argtypes = [i64, i64, i64, vp, vp, vp]; L.orc_csr_validate.restype = C.c_int
            L.orc_baseline_threads.argtypes = [C.c_int]; L.orc_baseline_threads.restype = C.c_int
            base_args = [i64, vp, vp, vp, C.POINTER(_Ilu), vp, vp, d, i64, C.POINTER(_Info)]
            L.orc_cg_csr_omp.argtypes = base_args; L.orc_cg_csr_omp.restype = C.c_int
            L.orc_bicgstab_csr_omp.argtypes = base_args; L.orc_bicgstab_csr_omp.restype = C.c_int
            _lib = L
    return _lib


def _vp(a):
    return None if a is None else C.c_void_p(a.ctypes.data)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


# ------------------------------------------------------------------ formats / classification
def rne(v: float, prec: int) -> float:
    return lib().orc_rne(float(v), int(prec))


def classify(v: float, loss_tol: float = 1e-15) -> int:
    return lib().orc_classify(float(v), float(loss_tol))


def fp16_bits(r: float) -> int:
    return lib().orc_fp16_bits(float(r))


def fp16_value(b: int) -> float:
    return lib().orc_fp16_value(int(b))


def e4m3_bits(r: float) -> int:
    return lib().orc_e4m3_bits(float(r))


def e4m3_value(b: int) -> float:
    return lib().orc_e4m3_value(int(b))


def csr_validate(n_rows, n_cols, rowptr, colidx, vals) -> int:
    rowptr = np.ascontiguousarray(rowptr, np.int64)
    colidx = np.ascontiguousarray(colidx, np.int32)
    vals = _f64(vals)
    return lib().orc_csr_validate(n_rows, n_cols, len(colidx), _vp(rowptr), _vp(colidx), _vp(vals))


# ------------------------------------------------------------------ tile format
CANONICAL = ("TileRowidx", "TileColidx", "TilePrec", "Floor", "TileNnz", "Nonrow", "ValOff",
             "TileRowPtr", "RowIndex", "CsrRowptr", "CsrColidx", "Val64", "Val32", "Val16", "Val8")


class Tiles:
    """The oracle's canonical tile matrix (SURVEY c-1), held in C memory."""

    def __init__(self, n_rows, n_cols, rowptr, colidx, vals, T=16, classify=True, loss_tol=1e-15):
        self._s = _Tiles()
        self.rowptr = np.ascontiguousarray(rowptr, np.int64)
        self.colidx = np.ascontiguousarray(colidx, np.int32)
        self.vals = _f64(vals)
        st = lib().orc_tiles_build(n_rows, n_cols, len(self.colidx), _vp(self.rowptr), _vp(self.colidx),
                                   _vp(self.vals), T, int(bool(classify)), loss_tol, C.byref(self._s))
        self.status = st
        if st != OK:
            raise OracleError(st)
        self.n_rows, self.n_cols, self.T = n_rows, n_cols, T

    def __del__(self):
        try:
            if getattr(self, "_s", None) is not None and _lib is not None:
                _lib.orc_tiles_free(C.byref(self._s))
        except Exception:
            pass

    @property
    def tilenum(self):
        return self._s.tilenum

    @property
    def rownum(self):
        return self._s.rownum

    @property
    def n_tile_rows(self):
        return self._s.n_tile_rows

    def arrays(self) -> dict:
        """Copies of the canonical arrays as numpy (the bit-exact export contract)."""
        s = self._s
        nt, nr, nz = s.tilenum, s.rownum, s.nnz

        def arr(ptr, n, dt):
            if n == 0 or not ptr:
                return np.zeros(0, dt)
            return np.ctypeslib.as_array(ptr, shape=(n,)).astype(dt, copy=True)

        return {
            "TileRowidx": arr(s.TileRowidx, nt, np.int32), "TileColidx": arr(s.TileColidx, nt, np.int32),
            "TilePrec": arr(s.TilePrec, nt, np.uint8), "Floor": arr(s.Floor, nt, np.uint8),
            "TileNnz": arr(s.TileNnz, nt + 1, np.int64), "Nonrow": arr(s.Nonrow, nt + 1, np.int64),
            "ValOff": arr(s.ValOff, nt, np.int64), "TileRowPtr": arr(s.TileRowPtr, s.n_tile_rows + 1, np.int64),
            "RowIndex": arr(s.RowIndex, nr, np.uint8), "CsrRowptr": arr(s.CsrRowptr, nr, np.uint8),
            "CsrColidx": arr(s.CsrColidx, nz, np.uint8),
            "Val64": arr(s.Val64, s.nval[0], np.float64), "Val32": arr(s.Val32, s.nval[1], np.float32),
            "Val16": arr(s.Val16, s.nval[2], np.uint16), "Val8": arr(s.Val8, s.nval[3], np.uint8),
        }

    def tile_value(self, t, a):
        return lib().orc_tile_value(C.byref(self._s), t, a)

    def stored_csr(self):
        """(rowptr, colidx, vals) of the stored (TilePrec-rounded) values, row-major."""
        col = np.empty(len(self.colidx), np.int32)
        val = np.empty(len(self.colidx), np.float64)
        lib().orc_tiles_stored_csr(C.byref(self._s), _vp(self.rowptr), _vp(col), _vp(val))
        return self.rowptr.copy(), col, val

    def tile_eff(self, level=None, range_guard=True):
        out = np.empty(self.tilenum, np.uint8)
        lv = None if level is None else np.ascontiguousarray(level, np.uint8)
        lib().orc_tile_eff(C.byref(self._s), _vp(lv), int(range_guard), _vp(out))
        return out

    def spmv(self, x, level=None, range_guard=True):
        """y = A~ x (Alg. 5); returns (y, counts[FP64,FP32,FP16,FP8,bypass])."""
        x = _f64(x)
        y = np.empty(self.n_rows, np.float64)
        counts = np.zeros(5, np.int64)
        lv = None if level is None else np.ascontiguousarray(level, np.uint8)
        lib().orc_spmv_tiles(C.byref(self._s), _vp(x), _vp(y), _vp(lv), int(range_guard), None, _vp(counts))
        return y, counts


    def sticky_state(self):
        """Fresh state of the sticky (P:237 literal) variant: cur_t = TilePrec_t and the working
        copy of every stored value in tile order (c-5 "sticky variant")."""
        return StickyState(self)

    def spmv_sticky(self, state, x, level, range_guard=True):
        """One SpMV of the sticky variant; lowers `state` in place.  Returns (y, counts)."""
        x = _f64(x)
        y = np.empty(self.n_rows, np.float64)
        counts = np.zeros(5, np.int64)
        lv = np.ascontiguousarray(level, np.uint8)
        lib().orc_spmv_tiles(C.byref(self._s), _vp(x), _vp(y), _vp(lv), int(range_guard),
                             C.cast(C.pointer(state._s), C.c_void_p), _vp(counts))
        return y, counts


class StickyState:
    def __init__(self, A: "Tiles"):
        arr = A.arrays()
        self.cur = arr["TilePrec"].copy()
        tn = arr["TileNnz"]
        self.wv = np.empty(max(int(tn[-1]), 1), np.float64)
        for t in range(A.tilenum):
            for a in range(int(tn[t + 1] - tn[t])):
                self.wv[tn[t] + a] = A.tile_value(t, a)
        self._s = _Sticky(self.cur.ctypes.data_as(C.POINTER(C.c_uint8)),
                          self.wv.ctypes.data_as(C.POINTER(C.c_double)))


class OracleError(RuntimeError):
    def __init__(self, status):
        super().__init__(f"oracle status {status}")
        self.status = status


def levels(v, T, th):
    v = _f64(v)
    th = _f64(th)
    out = np.empty((len(v) + T - 1) // T, np.uint8)
    lib().orc_levels(_vp(v), len(v), T, _vp(th), _vp(out))
    return out


def spmv_csr(rowptr, colidx, vals, x):
    rowptr = np.ascontiguousarray(rowptr, np.int64)
    colidx = np.ascontiguousarray(colidx, np.int32)
    vals, x = _f64(vals), _f64(x)
    n = len(rowptr) - 1
    y = np.empty(n, np.float64)
    lib().orc_spmv_csr(n, _vp(rowptr), _vp(colidx), _vp(vals), _vp(x), _vp(y))
    return y


# ------------------------------------------------------------------ dots and plans
class Plan:
    """Kernel-order reduction plan (SURVEY c-7): G CTAs, B threads, CTA g owns rows [R[g], R[g+1])."""

    def __init__(self, G, B, R, rank_ctas=None):
        """rank_ctas: CTA boundaries [0, G_0, G_0 + G_1, ..., G] of row-block ranks (each rank's
        CTAs own its rows): rank partials, summed in rank order from +0 (mf_oracle.c section 6)."""
        self.R = np.ascontiguousarray(R, np.int64)
        assert len(self.R) == G + 1 and B % 32 == 0
        self.Gr = None if rank_ctas is None else np.ascontiguousarray(rank_ctas, np.int32)
        if self.Gr is not None:
            assert self.Gr[0] == 0 and self.Gr[-1] == G and np.all(np.diff(self.Gr) >= 0)
        P = 0 if self.Gr is None else len(self.Gr) - 1
        gr = None if self.Gr is None else self.Gr.ctypes.data_as(C.POINTER(C.c_int32))
        self._s = _Plan(G, B, self.R.ctypes.data_as(C.POINTER(C.c_int64)), P, gr)
        self.G, self.B = G, B


def _plan_ref(plan):
    return None if plan is None else C.byref(plan._s)


def dot(u, v, plan: Plan | None = None) -> float:
    u, v = _f64(u), _f64(v)
    return lib().orc_dot(_vp(u), _vp(v), len(u), _plan_ref(plan))


# ------------------------------------------------------------------ ILU(0)
class ILU0:
    """ILU(0) factors.  rb_depth = 0: row-by-row substitution; d > 0: the recursive block
    SpTRSV of P:166 with d levels of splitting (mf_oracle.c rb_lower / rb_upper)."""
    def __init__(self, rowptr, colidx, vals, rb_depth: int = 0):
        self.rowptr = np.ascontiguousarray(rowptr, np.int64)
        self.colidx = np.ascontiguousarray(colidx, np.int32)
        vals = _f64(vals)
        self.n = len(self.rowptr) - 1
        self.lu = np.empty_like(vals)
        self.diag = np.empty(self.n, np.int64)
        st = lib().orc_ilu0(self.n, _vp(self.rowptr), _vp(self.colidx), _vp(vals), _vp(self.lu), _vp(self.diag))
        if st != OK:
            raise OracleError(st)
        self._s = _Ilu(self.n, self.rowptr.ctypes.data_as(C.POINTER(C.c_int64)),
                       self.colidx.ctypes.data_as(C.POINTER(C.c_int32)),
                       self.lu.ctypes.data_as(C.POINTER(C.c_double)),
                       self.diag.ctypes.data_as(C.POINTER(C.c_int64)), int(rb_depth))

    def apply(self, r):
        r = _f64(r)
        z = np.empty(self.n, np.float64)
        lib().orc_ilu_apply(C.byref(self._s), _vp(r), _vp(z))
        return z


# ------------------------------------------------------------------ solvers
def _opts(tol, max_iter, mode, switch_eps, switch_absolute, sticky, range_guard):
    # default eps = tol: the convergence threshold of P:174 is the stop tolerance of P:264
    # (reading R8)
    return _Opts(tol, max_iter, mode, tol if switch_eps is None else switch_eps,
                 int(switch_absolute), int(sticky), int(range_guard))


def _solve(fn, A: Tiles, b, x0, M, tol, max_iter, mode, switch_eps, switch_absolute, sticky,
           range_guard, plan, hist_cap):
    b = _f64(b)
    x = np.zeros(A.n_rows) if x0 is None else _f64(x0).copy()
    hist = np.full(hist_cap, np.nan)
    lc_cap = 2 * max_iter + 4
    lcounts = np.zeros((lc_cap, 5), np.int64)
    info = _Info()
    o = _opts(tol, max_iter, mode, switch_eps, switch_absolute, sticky, range_guard)
    st = fn(C.byref(A._s), None if M is None else C.byref(M._s), _vp(b), _vp(x), C.byref(o),
            _plan_ref(plan), _vp(hist), hist_cap, _vp(lcounts), lc_cap, C.byref(info))
    k = info.iterations
    return {"x": x, "status": st, "iterations": k, "converged": bool(info.converged),
            "rel_residual": info.rel_residual, "history": hist[: min(k + 1, hist_cap)],
            "level_counts": lcounts[: min(info.n_spmv, lc_cap)], "n_spmv": info.n_spmv}


def cg(A, b, x0=None, tol=1e-10, max_iter=1000, mode=MODE_DYNAMIC, switch_eps=None,
       switch_absolute=False, sticky=False, range_guard=True, plan=None, hist_cap=None, M=None):
    hist_cap = hist_cap or max_iter + 2
    return _solve(lib().orc_pcg, A, b, x0, M, tol, max_iter, mode, switch_eps, switch_absolute, sticky,
                  range_guard, plan, hist_cap)


def cg_single_reduction(A, b, x0=None, tol=1e-10, max_iter=1000, mode=MODE_DYNAMIC, switch_eps=None,
                        switch_absolute=False, sticky=False, range_guard=True, plan=None, hist_cap=None):
    """The one-reduction (Chronopoulos-Gear) CG variant, same options as cg()."""
    hist_cap = hist_cap or max_iter + 2
    L = lib()

    def fn(At, M, b_, x_, o, pl, h, hc, lc, lcc, info):
        return L.orc_cg_single_reduction(At, b_, x_, o, pl, h, hc, lc, lcc, info)
    return _solve(fn, A, b, x0, None, tol, max_iter, mode, switch_eps, switch_absolute, sticky, range_guard, plan,
                  hist_cap)


def bicgstab(A, b, x0=None, tol=1e-10, max_iter=1000, mode=MODE_DYNAMIC, switch_eps=None,
             switch_absolute=False, sticky=False, range_guard=True, plan=None, hist_cap=None, M=None):
    hist_cap = hist_cap or max_iter + 2
    return _solve(lib().orc_pbicgstab, A, b, x0, M, tol, max_iter, mode, switch_eps, switch_absolute,
                  sticky, range_guard, plan, hist_cap)


def cg_csr(rowptr, colidx, vals, b, x0=None, tol=1e-10, max_iter=1000):
    """Textbook FP64 CG on CSR, plain sequential dots (the CPU baseline)."""
    rowptr = np.ascontiguousarray(rowptr, np.int64)
    colidx = np.ascontiguousarray(colidx, np.int32)
    vals, b = _f64(vals), _f64(b)
    n = len(rowptr) - 1
    x = np.zeros(n) if x0 is None else _f64(x0).copy()
    hist = np.full(max_iter + 2, np.nan)
    info = _Info()
    st = lib().orc_cg_csr(n, _vp(rowptr), _vp(colidx), _vp(vals), _vp(b), _vp(x), tol, max_iter,
                          _vp(hist), max_iter + 2, C.byref(info))
    k = info.iterations
    return {"x": x, "status": st, "iterations": k, "converged": bool(info.converged),
            "rel_residual": info.rel_residual, "history": hist[: k + 1]}


def true_relres(rowptr, colidx, vals, b, x) -> float:
    rowptr = np.ascontiguousarray(rowptr, np.int64)
    colidx = np.ascontiguousarray(colidx, np.int32)
    vals, b, x = _f64(vals), _f64(b), _f64(x)
    return lib().orc_true_relres(len(rowptr) - 1, _vp(rowptr), _vp(colidx), _vp(vals), _vp(b), _vp(x))


def baseline_solve(kind, rowptr, colidx, vals, b, M=None, tol=1e-10, max_iter=1000, threads=0):
    """The CPU baseline of BASELINE.md section 7: textbook binary64 CSR CG ("cg") or BiCGSTAB
    ("bicgstab"), ILU(0)-preconditioned when M is an ILU0, OpenMP over `threads` host threads
    (0 = all in the affinity mask).  Returns the result dict plus the thread count used."""
    rowptr = np.ascontiguousarray(rowptr, np.int64)
    colidx = np.ascontiguousarray(colidx, np.int32)
    vals, b = _f64(vals), _f64(b)
    n = len(rowptr) - 1
    used = lib().orc_baseline_threads(int(threads) if threads else len(os.sched_getaffinity(0)))
    x = np.zeros(n)
    info = _Info()
    fn = lib().orc_cg_csr_omp if kind == "cg" else lib().orc_bicgstab_csr_omp
    st = fn(n, _vp(rowptr), _vp(colidx), _vp(vals), None if M is None else C.byref(M._s), _vp(b), _vp(x),
            float(tol), int(max_iter), C.byref(info))
    return {"x": x, "status": st, "iterations": info.iterations, "converged": bool(info.converged),
            "rel_residual": info.rel_residual, "threads": used}
