"""Pins for the two parts of the dynamic switch that round 1 left unpinned:

* the sticky variant (P:237 literal, SURVEY c-5 "sticky variant"): a tile lowered at one SpMV
  keeps its lowered working values; a further lowering rounds the CURRENT copy again
  (successive RNE), not the original value; bypass is never sticky;
* the threshold base tau ("the convergence threshold eps", stop test P:264 relative):
  tau = eps * ||v0||_2 with v0 the first SpMV input (CG: r0 = b; PCG: z0 = M^-1 r0;
  PBiCGSTAB: p^0 = M^-1 r0), eps = tol by default (reading R8).

Every expected value here is computed independently of the oracle: numpy float32/float16
casts, an E4M3 rounding written out below, the effective-precision rule of c-5 re-stated on
the exported canonical arrays, and numpy triangular solves for M^-1.
"""
import json
import math
import os

import numpy as np
import pytest

import workloads as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
FP64, FP32, FP16, FP8, BYP = 0, 1, 2, 3, 4


def e4m3(v: float) -> float:
    """Round-to-nearest-even to OCP E4M3FN (normal range only; values here are in [1, 2))."""
    a = abs(v)
    ex = math.floor(math.log2(a))
    q = 2.0 ** (ex - 3)
    return math.copysign(round(a / q) * q, v)      # python round(): half to even


def one_tile_row(values_by_col):
    """16 rows; row r has an entry in column 16*k + r for every tile column k listed."""
    ks = sorted(values_by_col)
    n = 16 * (max(ks) + 1)
    rowptr = np.zeros(n + 1, np.int64)
    rowptr[1:17] = np.arange(1, 17) * len(ks)
    rowptr[17:] = rowptr[16]
    cols = np.array([[16 * k + r for k in ks] for r in range(16)], np.int32).ravel()
    vals = np.array([[values_by_col[k] for k in ks] for r in range(16)]).ravel()
    return n, rowptr, cols, vals


def test_sticky_rounds_the_current_copy(orc):
    # v needs FP64 (2^-40 term).  RNE32(v) = 1.0625 + 2^-20; RNE16 of that = 1.0625, exactly the
    # E4M3 midpoint between 1.0 and 1.125 -> ties to even 1.0.  A single RNE8(v) gives 1.125.
    v = 1.0625 + 2.0 ** -20 + 2.0 ** -40
    w = 1.0 + 2.0 ** -30 + 2.0 ** -45            # second tile column, FP64 class
    n, rowptr, cols, vals = one_tile_row({0: v, 1: w})
    A = orc.Tiles(n, n, rowptr, cols, vals)
    arr = A.arrays()
    assert list(arr["TilePrec"]) == [FP64, FP64] and list(arr["Floor"]) == [FP8, FP8]
    v32 = float(np.float32(v))
    v16 = float(np.float16(v32))
    v8 = e4m3(v16)
    assert (v32, v16, v8) == (1.0625 + 2.0 ** -20, 1.0625, 1.0)
    assert e4m3(v) == 1.125 != v8                   # successive != single rounding
    x = np.zeros(n)
    x[:16] = 1.0
    x[16:] = 2.0 ** -3
    st = A.sticky_state()
    seq = [  # (level of segment 0, level of segment 1) -> expected (value used col 0, col 1)
        ((FP32, FP64), (v32, w)),
        ((FP16, BYP), (v16, None)),                 # col 1 bypassed: not sticky
        ((FP8, FP64), (v8, w)),                     # col 1 back at full precision
        ((FP64, FP32), (v8, float(np.float32(w)))),  # col 0 never rises again
        ((FP64, FP64), (v8, float(np.float32(w)))),
    ]
    for (l0, l1), (a0, a1) in seq:
        y, counts = A.spmv_sticky(st, x, np.array([l0, l1], np.uint8))
        # row chain fma(a1, 2^-3, fma(a0, 1, 0)): the product a1 * 2^-3 is exact -> one rounding
        want = a0 if a1 is None else a0 + a1 * 2.0 ** -3
        assert np.all(y[:16] == want), (l0, l1, y[0], want)
        assert counts[BYP] == (1 if a1 is None else 0)
    assert list(st.cur) == [FP8, FP32]
    # the per-iteration (default) reading at the same levels uses RNE8 of the stored value
    y, _ = A.spmv(x, np.array([FP8, BYP], np.uint8))
    assert np.all(y[:16] == e4m3(v))


def _fig7_matrix(g):
    n, T = g["n"], g["T"]
    rows, cols, vals = [], [], []
    k = 0
    for tr, tc, prec in g["tiles"]:
        for lr in range(T):
            for lc in range(T):
                k += 1
                v = 1.0 + (k % 7 + 1) / 7.0
                v = {0: v, 1: float(np.float32(v)), 2: float(np.float16(v)), 3: 1.0 + (k % 8) / 8.0}[prec]
                rows.append((tr - 1) * T + lr)
                cols.append((tc - 1) * T + lc)
                vals.append(v)
    order = np.lexsort((cols, rows))
    rows, cols, vals = np.array(rows)[order], np.array(cols)[order], np.array(vals)[order]
    rowptr = np.zeros(n + 1, np.int64)
    np.cumsum(np.bincount(rows, minlength=n), out=rowptr[1:])
    return rowptr, cols.astype(np.int32), vals


def test_fig7_replay_sticky_state(orc):
    """Fig. 7 driven through the oracle's own sticky SpMV: the in-place state lowers
    6, 8, 9 tiles at n, n+1, n+2 and 6 tiles are bypassed at n+3."""
    g = json.load(open(os.path.join(GOLDEN, "fig7.json")))
    rowptr, cols, vals = _fig7_matrix(g)
    A = orc.Tiles(g["n"], g["n"], rowptr, cols, vals, T=g["T"])
    tau = 3.0e-7
    th = [tau * 1e-3, tau * 1e-2, tau * 1e-1, tau]
    st = A.sticky_state()
    x = np.ones(g["n"])
    lowered, byp = [], []
    for seg in g["segment_values_over_tau"]:
        lv = orc.levels(np.repeat(np.array(seg) * tau, g["T"]), g["T"], th)
        before = st.cur.copy()
        _, counts = A.spmv_sticky(st, x, lv)
        lowered.append(int(np.sum(st.cur > before)))
        byp.append(int(counts[BYP]))
    assert lowered[1:4] == g["lowered"]
    assert lowered[0] == 0 and byp[-1] == g["bypassed_at_n_plus_3"] and byp[:-1] == [0, 0, 0, 0]


# ------------------------------------------------------------------------------ tau
def structured_rhs(n, seed):
    """Segments of 16 at magnitudes 10^-k (k = 0..15), random signs: the level pattern of the
    first SpMV is then sensitive to any rescaling of tau."""
    rng = np.random.default_rng(seed)
    k = rng.integers(0, 16, (n + 15) // 16)
    mag = np.repeat(10.0 ** -k.astype(float), 16)[:n]
    return mag * rng.uniform(1.0, 1.9, n) * rng.choice([-1.0, 1.0], n)


def expected_counts(arr, v0, tau):
    """c-5 restated: levels from max|v0| per segment, then e_t per tile (range guard on)."""
    n = len(v0)
    m = np.array([np.max(np.abs(v0[s:s + 16])) for s in range(0, n, 16)])
    th = [tau * 1e-3, tau * 1e-2, tau * 1e-1, tau]
    lev = np.where(m < th[0], BYP, np.where(m < th[1], FP8, np.where(m < th[2], FP16,
                   np.where(m < th[3], FP32, FP64))))
    lv = lev[arr["TileColidx"]]
    e = np.minimum(np.maximum(arr["TilePrec"], lv), arr["Floor"])
    e = np.where(lv == BYP, BYP, e)
    return np.bincount(e, minlength=5), lev


def _ilu_factors(M):
    n = M.n
    L, U = np.eye(n), np.zeros((n, n))
    for i in range(n):
        for k in range(M.rowptr[i], M.rowptr[i + 1]):
            j = M.colidx[k]
            if j < i:
                L[i, j] = M.lu[k]
            else:
                U[i, j] = M.lu[k]
    return L, U


@pytest.mark.parametrize("solver", ["cg", "bicgstab", "pcg", "pbicgstab"])
def test_tau_is_eps_times_norm_of_first_spmv_input(orc, solver):
    if solver in ("cg", "bicgstab"):
        A = W.make("C2", 16) if solver == "cg" else W.make("C3", 64)
    else:
        A = W.suitesparse_like(1024, seed=7, spd=solver == "pcg")
    T = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals, classify=True)
    arr = T.arrays()
    b = structured_rhs(A.n_rows, 11)
    M = None
    v0 = b
    if solver.startswith("p"):
        rp, ci, sv = T.stored_csr()
        M = orc.ILU0(rp, ci, sv)
        L, U = _ilu_factors(M)
        b = L @ (U @ b)          # so that v0 = M^-1 b carries the segment structure
        v0 = np.linalg.solve(U, np.linalg.solve(L, b))
    fn = orc.cg if solver in ("cg", "pcg") else orc.bicgstab
    tol = 1e-10
    r = fn(T, b, tol=tol, max_iter=1, M=M, mode=orc.MODE_DYNAMIC)
    got = r["level_counts"][0]
    tau = tol * math.sqrt(math.fsum(v0 * v0))
    want, lev = expected_counts(arr, v0, tau)
    assert np.array_equal(got, want), (got, want)
    # the pin discriminates: the level pattern moves under tau/sqrt(n) and under eps*100
    for alt in (tau / math.sqrt(A.n_rows), tau * 100.0):
        assert not np.array_equal(expected_counts(arr, v0, alt)[1], lev)
    # explicit eps and the literal absolute reading
    r2 = fn(T, b, tol=tol, max_iter=1, M=M, mode=orc.MODE_DYNAMIC, switch_eps=1e-6)
    assert np.array_equal(r2["level_counts"][0], expected_counts(arr, v0, 1e-6 * math.sqrt(math.fsum(v0 * v0)))[0])
    r3 = fn(T, b, tol=tol, max_iter=1, M=M, mode=orc.MODE_DYNAMIC, switch_eps=1e-9, switch_absolute=True)
    assert np.array_equal(r3["level_counts"][0], expected_counts(arr, v0, 1e-9)[0])
