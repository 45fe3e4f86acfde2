"""Pins for the convergent-element retrieval (Alg. 4), the effective tile precision
(Alg. 5 l.2-4), the mixed SpMV and the dot products.

Fig. 7 replay is the paper's own worked example; dense products with exact dyadic
arithmetic and math.fsum are the independent references for SpMV and dots.
"""
import json
import math
import os

import numpy as np
import pytest

import workloads as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _fig7_matrix(g):
    n, T = g["n"], g["T"]
    rows, cols, vals = [], [], []
    k = 0
    for tr, tc, prec in g["tiles"]:
        for lr in range(T):
            for lc in range(T):
                k += 1
                v = 1.0 + (k % 7 + 1) / 7.0          # in [1, 2): floor_t = FP8 for every tile
                v = {0: v, 1: float(np.float32(v)), 2: float(np.float16(v)), 3: 1.0 + (k % 8) / 8.0}[prec]
                rows.append((tr - 1) * T + lr)
                cols.append((tc - 1) * T + lc)
                vals.append(v)
    order = np.lexsort((cols, rows))
    rows, cols, vals = np.array(rows)[order], np.array(cols)[order], np.array(vals)[order]
    rowptr = np.zeros(n + 1, np.int64)
    np.cumsum(np.bincount(rows, minlength=n), out=rowptr[1:])
    return rowptr, cols.astype(np.int32), vals


def test_fig7_replay(orc):
    g = json.load(open(os.path.join(GOLDEN, "fig7.json")))
    rowptr, cols, vals = _fig7_matrix(g)
    A = orc.Tiles(g["n"], g["n"], rowptr, cols, vals, T=g["T"])
    arr = A.arrays()
    assert list(np.bincount(arr["TilePrec"], minlength=4)) == g["composition"]
    assert np.all(arr["Floor"] == orc.FP8)
    tau = 3.0e-7
    th = [tau * 1e-3, tau * 1e-2, tau * 1e-1, tau]
    prev = None
    cur_sticky = arr["TilePrec"].copy()
    lowered, bypassed = [], 0
    for it, seg in enumerate(g["segment_values_over_tau"]):
        p = np.repeat(np.array(seg) * tau, g["T"])
        lv = orc.levels(p, g["T"], th)
        e = A.tile_eff(lv)
        if prev is not None:
            nonbyp = (e != orc.BYPASS) & (prev != orc.BYPASS)
            lowered.append(int(np.sum(nonbyp & (e > prev))))
        # sticky reading: cur <- min_prec(cur, e) never rises; same counts on this example
        cur_sticky = np.where(e == orc.BYPASS, cur_sticky, np.maximum(cur_sticky, e))
        prev = e
        bypassed = int(np.sum(e == orc.BYPASS))
    assert lowered[:3] == g["lowered"]
    assert bypassed == g["bypassed_at_n_plus_3"]


def test_levels_interval_boundaries(orc):
    """P:174 half-open intervals: a value exactly at a threshold takes the higher precision."""
    th = np.array([1e-3, 1e-2, 1e-1, 1.0])
    cases = [(0.0, 4), (0.99e-3, 4), (1e-3, 3), (0.99e-2, 3), (1e-2, 2), (0.99e-1, 2),
             (1e-1, 1), (0.99, 1), (1.0, 0), (5.0, 0)]
    for v, lv in cases:
        for s in (1, -1):                  # |p| (reading R7)
            seg = np.zeros(16)
            seg[5] = s * v
            assert orc.levels(seg, 16, th)[0] == lv, (v, s)
    seg = np.zeros(16)
    seg[3] = np.nan
    assert orc.levels(seg, 16, th)[0] == orc.FP64
    # ragged tail: the last segment uses the elements that exist
    v = np.concatenate([np.full(16, 5.0), np.full(3, 1e-5)])
    assert list(orc.levels(v, 16, th)) == [0, 4]


def test_effective_precision_rule(orc):
    """e_t = bypass | max_prec(floor, min_prec(TilePrec, level)) over all combinations."""
    rows = np.arange(16)
    vals_by_prec = {0: 1 + 1 / 7, 1: float(np.float32(1 + 1 / 7)), 2: float(np.float16(1 + 1 / 7)), 3: 1.5}
    for tp in range(4):
        for small in ((False, True) if tp < 3 else (False,)):
            # small: 2^-10 scale keeps the class but leaves the E4M3 normal range -> floor FP16
            v = vals_by_prec[tp] * (2.0 ** -10 if small else 1.0)
            rp = np.arange(17, dtype=np.int64)
            A = orc.Tiles(16, 16, rp, rows.astype(np.int32), np.full(16, v))
            arr = A.arrays()
            f = arr["Floor"][0]
            assert arr["TilePrec"][0] == tp
            assert f == (max(tp, 2) if small else 3)
            for lv in range(5):
                e = A.tile_eff(np.array([lv], np.uint8))[0]
                e_noguard = A.tile_eff(np.array([lv], np.uint8), range_guard=False)[0]
                if lv == 4:
                    assert e == 4 and e_noguard == 4
                else:
                    assert e_noguard == max(tp, lv)
                    assert e == min(max(tp, lv), f)


def _dyadic_mixed_matrix(seed, n=48):
    """Values whose roundings are known and whose products/sums are exact in binary64:
    magnitudes 2^k * {1.5+2^-8+2^-12+2^-30 (FP64 class), 1.5+2^-8+2^-12 (FP32), 1.5+2^-8 (FP16),
    1.5 (FP8)}.  RNE32 drops 2^-30, RNE16 drops 2^-12, E4M3 keeps 1.5."""
    rng = np.random.default_rng(seed)
    M = rng.random((n, n)) < 0.2
    np.fill_diagonal(M, True)
    rows, cols = np.nonzero(M)
    base = np.array([1.5 + 2.0 ** -8 + 2.0 ** -12 + 2.0 ** -30, 1.5 + 2.0 ** -8 + 2.0 ** -12, 1.5 + 2.0 ** -8, 1.5])
    v = base[rng.integers(0, 4, rows.size)] * np.exp2(rng.integers(-3, 4, rows.size)) * rng.choice([-1, 1], rows.size)
    rowptr = np.zeros(n + 1, np.int64)
    np.cumsum(np.bincount(rows, minlength=n), out=rowptr[1:])
    return rowptr, cols.astype(np.int32), v


def _round_indep(v, e):
    """Independent rounding of the dyadic test values (numpy casts; E4M3 by construction)."""
    if e == 0:
        return v
    if e == 1:
        return float(np.float32(v))
    if e == 2:
        return float(np.float16(v))
    a = abs(v)
    ex = math.floor(math.log2(a))
    q = 2.0 ** (ex - 3)
    return math.copysign(round(a / q) * q, v)   # python round() is half-to-even


@pytest.mark.parametrize("seed", range(6))
def test_mixed_spmv_exact_vs_dense(orc, seed):
    rowptr, cols, vals = _dyadic_mixed_matrix(seed)
    n = len(rowptr) - 1
    A = orc.Tiles(n, n, rowptr, cols, vals, T=16)
    arr = A.arrays()
    rng = np.random.default_rng(100 + seed)
    x = np.exp2(rng.integers(-2, 3, n).astype(float)) * rng.choice([-1, 1], n)
    level = rng.integers(0, 5, (n + 15) // 16).astype(np.uint8)
    e = A.tile_eff(level)
    rp, ci, sv = A.stored_csr()
    tile_of = {(arr["TileRowidx"][t], arr["TileColidx"][t]): t for t in range(A.tilenum)}
    D = np.zeros((n, n))
    for i in range(n):
        for k in range(rp[i], rp[i + 1]):
            t = tile_of[(i // 16, ci[k] // 16)]
            if e[t] != orc.BYPASS:
                D[i, ci[k]] = _round_indep(sv[k], e[t])
    y, counts = A.spmv(x, level)
    assert np.array_equal(y, D @ x)          # exact: every product and partial sum is dyadic-exact
    assert counts.sum() == A.tilenum and list(counts) == [int(np.sum(e == q)) for q in range(5)]


@pytest.mark.parametrize("seed", range(4))
def test_tile_spmv_equals_csr_row_chain(orc, seed):
    """Two different traversals (tile walk vs CSR row walk) of the same per-row fma chain are
    bit-identical for arbitrary binary64 values (all-FP64 tiles)."""
    A = W.random_csr(100, 100, 0.08, seed, values="f64")
    T = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals, classify=False)
    x = np.random.default_rng(seed).standard_normal(100)
    y, _ = T.spmv(x)
    assert np.array_equal(y, orc.spmv_csr(A.rowptr, A.colidx, A.vals, x))
    assert np.allclose(y, A.dense() @ x, rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("n,G,B", [(1000, 1, 32), (5000, 7, 64), (100000, 148, 1024), (33, 3, 32)])
def test_dot_plan_vs_fsum(orc, n, G, B):
    rng = np.random.default_rng(n)
    u, v = rng.standard_normal(n), rng.standard_normal(n)
    R = (np.linspace(0, n, G + 1) // 16 * 16).astype(np.int64)
    R[-1] = n
    plan = orc.Plan(G, B, R)
    exact = math.fsum(u * v)
    scale = np.sum(np.abs(u * v))
    eps = 2.0 ** -53
    for p in (None, plan):
        d = orc.dot(u, v, p)
        assert abs(d - exact) <= 2 * n * eps * scale
    # the plan is a reordering only: exact inputs give exact sums in any order
    ui, vi = np.round(u * 8), np.round(v * 8)
    assert orc.dot(ui, vi, plan) == orc.dot(ui, vi) == float(np.dot(ui, vi))
