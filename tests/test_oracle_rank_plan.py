"""Pins of the oracle's rank-partitioned reduction plan (mf_oracle.c section 6, row-block ranks;
the multi-GPU reading of DESIGN.md: every dot is the sum, in rank order from +0, of the rank
partials, each the single-launch tree over that rank's CTAs).

What fixes it other than the oracle itself:
  * exact inputs (small integers): any summation order gives the exact dot (np.dot);
  * a rank partial is the dot of the rank's rows under that rank's own plan (rows re-based),
    and the total composes them left to right from +0 -- the decomposition is checked with
    three ranks whose partials are 1e16, 1, -1e16: rank order gives 0 (1e16 + 1 rounds to
    1e16), while one tree over all CTAs pairs 1e16 with -1e16 first and gives 1;
  * one rank is the single-launch plan plus a leading +0 (bit-identical for nonzero sums)."""
import math

import numpy as np
import pytest


def _plan_for(orc, bounds, ctas_per_rank, B):
    """Global plan of ranks with row blocks `bounds`, each split evenly into its CTAs."""
    R, Gr = [], [0]
    for k in range(len(bounds) - 1):
        rb, re = bounds[k], bounds[k + 1]
        g = ctas_per_rank[k]
        r = np.linspace(rb, re, g + 1).astype(np.int64)
        R.extend(r[:-1].tolist())
        Gr.append(Gr[-1] + g)
    R.append(bounds[-1])
    return orc.Plan(Gr[-1], B, np.array(R, np.int64), rank_ctas=Gr), R, Gr


def test_rank_plan_exact_on_integers(orc):
    rng = np.random.default_rng(3)
    n = 5000
    u, v = np.round(rng.standard_normal(n) * 16), np.round(rng.standard_normal(n) * 16)
    plan, _, _ = _plan_for(orc, [0, 1200, 3000, 5000], [3, 5, 2], 64)
    assert orc.dot(u, v, plan) == float(np.dot(u, v))


def test_rank_plan_error_bound(orc):
    rng = np.random.default_rng(4)
    n = 20000
    u, v = rng.standard_normal(n), rng.standard_normal(n)
    plan, _, _ = _plan_for(orc, [0, 7000, 12000, 20000], [4, 4, 4], 128)
    d = orc.dot(u, v, plan)
    assert abs(d - math.fsum(u * v)) <= 2 * n * 2.0 ** -53 * np.sum(np.abs(u * v))


def test_rank_plan_composes_rank_partials_in_order(orc):
    n = 96
    bounds = [0, 32, 64, 96]
    u = np.zeros(n)
    v = np.ones(n)
    u[5], u[40], u[70] = 1e16, 1.0, -1e16          # one value per rank
    plan, R, Gr = _plan_for(orc, bounds, [1, 1, 1], 32)
    assert orc.dot(u, v, plan) == 0.0               # ((+0 + 1e16) + 1) + -1e16
    single = orc.Plan(3, 32, np.array(R, np.int64))
    assert orc.dot(u, v, single) == 1.0             # tree32 over the 3 CTAs: (1e16 + -1e16) + 1
    # general decomposition: rank q's partial is the dot of its rows under its own plan
    rng = np.random.default_rng(5)
    n = 3000
    bounds = [0, 1000, 2200, 3000]
    u, v = rng.standard_normal(n), rng.standard_normal(n)
    plan, R, Gr = _plan_for(orc, bounds, [3, 2, 4], 64)
    tot = 0.0
    for k in range(3):
        rk = np.array(R[Gr[k]:Gr[k + 1]] + [bounds[k + 1]], np.int64) - bounds[k]
        pk = orc.Plan(Gr[k + 1] - Gr[k], 64, rk)
        tot = tot + orc.dot(u[bounds[k]:bounds[k + 1]], v[bounds[k]:bounds[k + 1]], pk)
    assert orc.dot(u, v, plan) == tot


@pytest.mark.parametrize("G,B", [(1, 32), (7, 256), (148, 512)])
def test_one_rank_is_the_single_launch_plan(orc, G, B):
    rng = np.random.default_rng(G)
    n = 40000
    u, v = rng.standard_normal(n), rng.standard_normal(n)
    R = (np.linspace(0, n, G + 1) // 16 * 16).astype(np.int64)
    R[-1] = n
    one = orc.Plan(G, B, R, rank_ctas=[0, G])
    assert orc.dot(u, v, one) == orc.dot(u, v, orc.Plan(G, B, R))


def test_rank_plan_cg_converges_like_single_plan(orc):
    import workloads as W
    A = W.make("C2", 16)
    b = W.rhs_ones(A)
    T = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
    plan, _, _ = _plan_for(orc, [0, 1024, 2560, 4096], [4, 4, 4], 256)
    r1 = orc.cg(T, b, mode=2, plan=plan, max_iter=500)
    r0 = orc.cg(T, b, mode=2, max_iter=500)
    assert r1["converged"] and r0["converged"]
    assert abs(r1["iterations"] - r0["iterations"]) <= 2
    assert np.max(np.abs(r1["x"] - r0["x"])) < 1e-8
