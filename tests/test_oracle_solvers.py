"""Pins for the oracle's CG / BiCGSTAB (Alg. 1-2), PCG / PBiCGSTAB with ILU(0)
 and the precision modes.

Independent references: numpy.linalg.solve, CG finite termination on k distinct eigenvalues
and within n steps, residual orthogonality and A-orthogonality of the search directions, the
recurrence-vs-true residual gap, x* = 1 for b = A*1, exact LU for tridiagonal ILU(0).
"""
import numpy as np
import pytest

import workloads as W


def csr_from_dense(D):
    rows, cols = np.nonzero(D)
    rowptr = np.zeros(D.shape[0] + 1, np.int64)
    np.cumsum(np.bincount(rows, minlength=D.shape[0]), out=rowptr[1:])
    return W.CSR(D.shape[0], D.shape[1], rowptr, cols.astype(np.int32), D[rows, cols].astype(np.float64))


def tiles(orc, A, classify=False):
    return orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals, classify=classify)


def rand_spd(n, seed, cond=50.0):
    rng = np.random.default_rng(seed)
    Q, _ = np.linalg.qr(rng.standard_normal((n, n)))
    ev = np.geomspace(1.0, cond, n)
    return (Q * ev) @ Q.T


@pytest.mark.parametrize("n,seed", [(8, 0), (30, 1), (64, 2)])
def test_cg_matches_dense_solve(orc, n, seed):
    D = rand_spd(n, seed)
    A = csr_from_dense(D)
    b = np.random.default_rng(seed).standard_normal(n)
    r = orc.cg(tiles(orc, A), b, tol=1e-12, mode=orc.MODE_FP64)
    assert r["converged"] and r["status"] == 0
    x = np.linalg.solve(D, b)
    assert np.linalg.norm(r["x"] - x) / np.linalg.norm(x) < 50 * 1e-10
    assert r["iterations"] <= 3 * n


@pytest.mark.parametrize("k", [1, 2, 3, 5])
def test_cg_finite_termination_k_distinct_eigenvalues(orc, k):
    n = 40
    d = np.array([1.0, 2.5, 4.0, 7.0, 11.0])[:k][np.arange(n) % k]
    A = csr_from_dense(np.diag(d))
    b = np.random.default_rng(k).standard_normal(n)
    r = orc.cg(tiles(orc, A), b, tol=1e-13, mode=orc.MODE_FP64)
    assert r["converged"] and r["iterations"] <= k


@pytest.mark.parametrize("n", [4, 9, 16])
def test_cg_terminates_within_n_steps(orc, n):
    D = rand_spd(n, n, cond=10.0)
    A = csr_from_dense(D)
    b = np.ones(n)
    r = orc.cg(tiles(orc, A), b, tol=1e-10, mode=orc.MODE_FP64)
    assert r["converged"] and r["iterations"] <= n


def _iterates(orc, solver, T, b, steps, **kw):
    return [solver(T, b, max_iter=j, tol=0.0, **kw)["x"] for j in range(steps + 1)]


def test_cg_orthogonality_invariants(orc):
    """Residuals r_i = b - A x_i are mutually orthogonal; directions x_{j+1}-x_j are A-conjugate."""
    A = W.poisson2d(12)
    D = A.dense()
    T = tiles(orc, A)
    b = W.rhs_ones(A) + np.random.default_rng(0).standard_normal(A.n_rows) * 0.1
    xs = _iterates(orc, orc.cg, T, b, 8, mode=orc.MODE_FP64)
    R = np.array([b - D @ x for x in xs])
    G = R @ R.T
    nr = np.sqrt(np.diag(G))
    off = np.abs(G / np.outer(nr, nr) - np.eye(len(xs)))
    assert off.max() < 1e-10
    P = np.diff(np.array(xs), axis=0)
    GA = P @ D @ P.T
    na = np.sqrt(np.diag(GA))
    assert np.abs(GA / np.outer(na, na) - np.eye(len(P))).max() < 1e-10


@pytest.mark.parametrize("solver", ["cg", "bicgstab"])
def test_recurrence_gap(orc, solver):
    """The recorded recurrence residual relres_j equals the true ||b - A x_j||/||b|| to 1e-12."""
    A = W.poisson2d(24) if solver == "cg" else W.convdiff2d(24)
    T = tiles(orc, A)
    b = W.rhs_ones(A)
    fn = getattr(orc, solver)
    full = fn(T, b, mode=orc.MODE_FP64, max_iter=200)
    for j in (1, 5, 10, 20):
        rj = fn(T, b, mode=orc.MODE_FP64, max_iter=j, tol=0.0)
        true = orc.true_relres(A.rowptr, A.colidx, A.vals, b, rj["x"])
        assert abs(full["history"][j] - true) < 1e-12
        assert rj["history"][j] == full["history"][j]


def test_cg_poisson_solution_is_ones(orc):
    A = W.poisson2d(64)
    r = orc.cg(tiles(orc, A, classify=True), W.rhs_ones(A))
    assert r["converged"] and r["iterations"] == 135
    assert np.max(np.abs(r["x"] - 1.0)) < 1e-8


@pytest.mark.parametrize("n,seed", [(10, 0), (40, 1), (64, 3)])
def test_bicgstab_matches_dense_solve(orc, n, seed):
    rng = np.random.default_rng(seed)
    D = rng.standard_normal((n, n)) * (rng.random((n, n)) < 0.3) + np.diag(np.full(n, 6.0))
    A = csr_from_dense(D)
    b = rng.standard_normal(n)
    r = orc.bicgstab(tiles(orc, A), b, tol=1e-12, mode=orc.MODE_FP64)
    assert r["converged"] and r["status"] == 0
    x = np.linalg.solve(D, b)
    assert np.linalg.norm(r["x"] - x) / np.linalg.norm(x) < 1e-9


def test_bicgstab_one_step_on_scaled_identity(orc):
    A = csr_from_dense(np.eye(20) * 3.0)
    b = np.random.default_rng(0).standard_normal(20)
    r = orc.bicgstab(tiles(orc, A), b, tol=1e-14, mode=orc.MODE_FP64)
    assert r["converged"] and r["iterations"] <= 1
    assert np.allclose(r["x"], b / 3.0, rtol=1e-15, atol=0)


@pytest.mark.parametrize("name,scale,solver", [("C1", 32, "cg"), ("C3", 64, "bicgstab")])
def test_static_mixed_equals_fp64_on_exact_values(orc, name, scale, solver):
    """Poisson / C3-Q00 values are exact at their tile precision: static mixed == FP64 bit for
    bit (exact upcast + identical fma chains).  C3 has FP64-class tiles, where stored == v."""
    A = W.make(name, scale)
    b = W.rhs_ones(A)
    fn = getattr(orc, solver)
    r64 = fn(tiles(orc, A, classify=False), b, mode=orc.MODE_FP64, max_iter=3000)
    rst = fn(tiles(orc, A, classify=True), b, mode=orc.MODE_STATIC, max_iter=3000)
    assert r64["iterations"] == rst["iterations"]
    assert np.array_equal(r64["history"], rst["history"]) and np.array_equal(r64["x"], rst["x"])


@pytest.mark.parametrize("solver", ["cg", "bicgstab"])
def test_dynamic_with_zero_eps_equals_static(orc, solver):
    A = W.make("C2", 16) if solver == "cg" else W.make("C3", 48)
    T = tiles(orc, A, classify=True)
    b = W.rhs_ones(A)
    fn = getattr(orc, solver)
    st = fn(T, b, mode=orc.MODE_STATIC, max_iter=2000)
    dy = fn(T, b, mode=orc.MODE_DYNAMIC, switch_eps=0.0, max_iter=2000)
    assert np.array_equal(st["history"], dy["history"]) and np.array_equal(st["x"], dy["x"])
    sk = fn(T, b, mode=orc.MODE_DYNAMIC, switch_eps=0.0, sticky=True, max_iter=2000)
    assert np.array_equal(st["x"], sk["x"])


def test_kernel_order_plan_changes_only_rounding(orc):
    A = W.poisson2d(64)
    T = tiles(orc, A, classify=True)
    b = W.rhs_ones(A)
    R = np.array([0, 1024, 2048, 3072, 4096], np.int64)
    plain = orc.cg(T, b, mode=orc.MODE_FP64)
    planned = orc.cg(T, b, mode=orc.MODE_FP64, plan=orc.Plan(4, 256, R))
    assert plain["iterations"] == planned["iterations"]
    h0, h1 = plain["history"], planned["history"]
    assert np.max(np.abs(h0 - h1) / h0) < 1e-8


def test_dynamic_mixed_converges_and_reports_levels(orc):
    A = W.make("C2", 32)
    T = tiles(orc, A, classify=True)
    b = W.rhs_ones(A)
    dy = orc.cg(T, b, mode=orc.MODE_DYNAMIC)
    assert dy["converged"]
    lc = dy["level_counts"]
    assert lc.shape == (dy["iterations"], 5) and np.all(lc.sum(1) == T.tilenum)
    assert orc.true_relres(A.rowptr, A.colidx, A.vals, b, dy["x"]) < 1e-9
    sk = orc.cg(T, b, mode=orc.MODE_DYNAMIC, sticky=True)
    assert sk["converged"]


def test_cg_breakdown_and_edge_cases(orc):
    A = csr_from_dense(np.diag(np.array([1.0, -1.0, 2.0, -3.0])))
    r = orc.cg(tiles(orc, A), np.ones(4), mode=orc.MODE_FP64)
    assert r["status"] == orc.ERR_BREAKDOWN
    B = W.poisson2d(8)
    r0 = orc.cg(tiles(orc, B), np.zeros(64), x0=np.ones(64))
    assert r0["converged"] and r0["iterations"] == 0 and np.all(r0["x"] == 0)
    rm = orc.cg(tiles(orc, B), W.rhs_ones(B), max_iter=3)
    assert rm["status"] == 0 and not rm["converged"] and rm["iterations"] == 3
    x0 = np.random.default_rng(0).standard_normal(64)
    rx = orc.cg(tiles(orc, B), W.rhs_ones(B), x0=x0)
    assert rx["converged"] and np.max(np.abs(rx["x"] - 1)) < 1e-8


def _lu_dense(M, n):
    L, U = np.eye(n), np.zeros((n, n))
    for i in range(n):
        for k in range(M.rowptr[i], M.rowptr[i + 1]):
            j = M.colidx[k]
            if j < i:
                L[i, j] = M.lu[k]
            else:
                U[i, j] = M.lu[k]
    return L, U


def test_ilu0_tridiagonal_is_exact_lu(orc):
    n = 50
    D = np.diag(np.full(n, 4.0)) + np.diag(np.full(n - 1, -1.3), 1) + np.diag(np.full(n - 1, -0.7), -1)
    A = csr_from_dense(D)
    M = orc.ILU0(A.rowptr, A.colidx, A.vals)
    L, U = _lu_dense(M, n)
    assert np.allclose(L @ U, D, rtol=0, atol=1e-14)
    v = np.random.default_rng(0).standard_normal(n)
    assert np.allclose(M.apply(D @ v), v, rtol=0, atol=1e-13)
    Dsym = np.diag(np.full(n, 4.0)) + np.diag(np.full(n - 1, -1.0), 1) + np.diag(np.full(n - 1, -1.0), -1)
    S = csr_from_dense(Dsym)
    Ms = orc.ILU0(S.rowptr, S.colidx, S.vals)
    r = orc.cg(tiles(orc, S), Dsym @ np.ones(n), M=Ms, mode=orc.MODE_FP64, tol=1e-12)
    assert r["converged"] and r["iterations"] <= 1


def test_ilu0_matches_a_on_pattern(orc):
    A = W.suitesparse_like(512, seed=3, spd=False)
    M = orc.ILU0(A.rowptr, A.colidx, A.vals)
    L, U = _lu_dense(M, A.n_rows)
    LU = L @ U
    rows = np.repeat(np.arange(A.n_rows), np.diff(A.rowptr))
    scale = np.abs(A.vals).max()
    assert np.max(np.abs(LU[rows, A.colidx] - A.vals)) < 1e-12 * scale


def test_ilu0_zero_pivot(orc):
    # explicit zero on the diagonal of row 0
    A = W.CSR(2, 2, np.array([0, 2, 4], np.int64), np.array([0, 1, 0, 1], np.int32), np.array([0.0, 1, 1, 2]))
    with pytest.raises(orc.OracleError) as e:
        orc.ILU0(A.rowptr, A.colidx, A.vals)
    assert e.value.status == orc.ERR_ZERO_PIVOT


@pytest.mark.parametrize("spd", [True, False])
def test_preconditioned_solvers_match_dense(orc, spd):
    A = W.suitesparse_like(2048, seed=5, spd=spd)
    T = tiles(orc, A, classify=True)
    rp, ci, sv = T.stored_csr()
    M = orc.ILU0(rp, ci, sv)
    b = W.rhs_ones(A)
    fn = orc.cg if spd else orc.bicgstab
    rp_ = fn(T, b, M=M, mode=orc.MODE_STATIC)
    ru = fn(T, b, mode=orc.MODE_STATIC)
    assert rp_["converged"] and rp_["iterations"] <= ru["iterations"]
    Ds = W.CSR(A.n_rows, A.n_cols, rp, ci, sv).dense()
    x = np.linalg.solve(Ds, b)
    assert np.linalg.norm(rp_["x"] - x) / np.linalg.norm(x) < 1e-8
    dyn = fn(T, b, M=M, mode=orc.MODE_DYNAMIC)
    assert dyn["converged"]


# ------------------------------------------------------------------ single-reduction CG (f4)
@pytest.mark.parametrize("n,seed", [(8, 0), (30, 1), (64, 2)])
def test_cg_single_reduction_matches_dense_solve(orc, n, seed):
    D = rand_spd(n, seed)
    A = csr_from_dense(D)
    b = np.random.default_rng(seed).standard_normal(n)
    r = orc.cg_single_reduction(tiles(orc, A), b, tol=1e-12, mode=orc.MODE_FP64)
    assert r["converged"] and r["status"] == 0
    x = np.linalg.solve(D, b)
    assert np.linalg.norm(r["x"] - x) / np.linalg.norm(x) < 50 * 1e-10


def test_cg_single_reduction_finite_termination(orc):
    """k distinct eigenvalues: the Krylov method ends in k iterations (exact-arithmetic identity
    with Alg. 1: same iterates, the recurrences only reorder the dots)."""
    n, k = 64, 4
    d = np.repeat(np.array([1.0, 2.0, 5.0, 9.0]), n // k)
    A = W.CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32), d)
    r = orc.cg_single_reduction(tiles(orc, A), np.ones(n), tol=1e-12, mode=orc.MODE_FP64)
    assert r["converged"] and r["iterations"] <= k
    assert np.allclose(r["x"], 1.0 / d, rtol=1e-11)


@pytest.mark.parametrize("name,scale", [("C1", 64), ("C2", 16)])
def test_cg_single_reduction_tracks_classic_cg(orc, name, scale):
    """Same Krylov iterates as Alg. 1 up to rounding: residual histories agree to ~1e-6 relative
    over the first iterations, iteration counts within 2%, same solution (x* = 1)."""
    A = W.make(name, scale)
    b = W.rhs_ones(A)
    T = tiles(orc, A, classify=True)
    rc = orc.cg(T, b, mode=orc.MODE_FP64)
    rs = orc.cg_single_reduction(T, b, mode=orc.MODE_FP64)
    assert rc["converged"] and rs["converged"]
    assert abs(rs["iterations"] - rc["iterations"]) <= max(2, rc["iterations"] // 50)
    m = 20
    assert np.max(np.abs(rs["history"][:m] - rc["history"][:m]) / rc["history"][:m]) < 1e-6
    assert np.max(np.abs(rs["x"] - 1.0)) < 1e-8
    dy = orc.cg_single_reduction(T, b, mode=orc.MODE_DYNAMIC)
    assert dy["converged"] and dy["n_spmv"] == dy["iterations"] + 1
