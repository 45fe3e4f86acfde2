"""Pins for the oracle's recursive block SpTRSV (reading R27).

P:166: "we recursively divide a triangular matrix into two smaller triangular blocks and one
square block.  The SpTRSV operation is utilized for the triangular blocks, and SpMV is applied to
the square blocks."  The recursion only regroups the sums of the substitution, so:
  * on integer triangular systems whose every partial sum is an exact binary64 integer the
    result must equal the exact solution (computed here in Python integers, no floating point);
  * on general systems it must agree with a dense LU solve (numpy) within the forward-error
    bound of a triangular solve;
  * depth 0 is the row-by-row substitution (bit for bit).
A dropped square block, a wrong column range (c >= lo / c < mid / c < hi), a wrong sign or a
missing division by u_ii fails the integer pins.
"""
import numpy as np
import pytest

import workloads as W


def _int_factors(n, seed, per_row=3):
    """Pattern of a random sparse matrix with diagonal; ILU0 object whose lu is then overwritten
    with integer L (unit) / U (diagonal +-1) entries.  Returns (M, L, U) with L, U as int dicts."""
    rng = np.random.default_rng(seed)
    rows = []
    for i in range(n):
        cols = set(rng.choice(n, size=min(per_row, n), replace=False).tolist()) | {i}
        rows.append(sorted(cols))
    rp = np.zeros(n + 1, np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    ci = np.array([c for r in rows for c in r], np.int32)
    vals = np.where(ci == np.repeat(np.arange(n), np.diff(rp)), 10.0, 0.5)   # valid pivots
    return rp, ci, vals, rng


def _exact_solve(n, rp, ci, lu, diag, r):
    """Python-integer forward (unit L) then backward (U) substitution."""
    y = [0] * n
    for i in range(n):
        acc = int(r[i])
        for k in range(rp[i], diag[i]):
            acc -= int(lu[k]) * y[ci[k]]
        y[i] = acc
    z = [0] * n
    for i in range(n - 1, -1, -1):
        acc = y[i]
        for k in range(diag[i] + 1, rp[i + 1]):
            acc -= int(lu[k]) * z[ci[k]]
        d = int(lu[diag[i]])
        assert acc % d == 0
        z[i] = acc // d
    return y, z


@pytest.mark.parametrize("n,seed,depth", [(77, 1, 1), (77, 1, 3), (160, 2, 2), (160, 2, 6), (301, 3, 4), (301, 3, 30)])
def test_rb_integer_exact(orc, n, seed, depth):
    rp, ci, vals, rng = _int_factors(n, seed)
    M = orc.ILU0(rp, ci, vals, rb_depth=depth)
    diag = M.diag
    for attempt in range(50):
        lu = rng.choice(np.array([-1.0, 1.0, 2.0, -2.0, 0.0]), p=[0.15, 0.15, 0.05, 0.05, 0.6], size=len(ci))
        lu[diag] = rng.choice(np.array([1.0, -1.0]), size=n)
        r = rng.integers(-3, 4, size=n).astype(np.float64)
        y, z = _exact_solve(n, rp, ci, lu, diag, r)
        if max(abs(v) for v in y + z) < 2 ** 40:     # every partial sum exact in binary64
            break
    else:
        pytest.skip("no bounded integer system for this seed")
    M.lu[:] = lu
    got = M.apply(r)
    assert np.array_equal(got, np.array(z, dtype=np.float64))
    M0 = orc.ILU0(rp, ci, vals, rb_depth=0)
    M0.lu[:] = lu
    assert np.array_equal(M0.apply(r), got)


@pytest.mark.parametrize("depth", [0, 1, 2, 5, 40])
def test_rb_matches_dense_lu(orc, depth):
    A = W.suitesparse_like(512, seed=11, spd=False)
    M = orc.ILU0(A.rowptr, A.colidx, A.vals, rb_depth=depth)
    n = A.n_rows
    L = np.eye(n)
    U = np.zeros((n, n))
    for i in range(n):
        for k in range(A.rowptr[i], A.rowptr[i + 1]):
            c = A.colidx[k]
            if c < i:
                L[i, c] = M.lu[k]
            else:
                U[i, c] = M.lu[k]
    r = np.random.default_rng(4).standard_normal(n)
    z = M.apply(r)
    ref = np.linalg.solve(U, np.linalg.solve(L, r))
    # forward error of two triangular solves: small multiple of n * u * cond (diagonally
    # dominant factors here: cond ~ 1)
    assert np.max(np.abs(z - ref)) <= 1e-12 * np.max(np.abs(ref))


def test_rb_depth0_is_substitution_bitwise(orc):
    A = W.suitesparse_like(1024, seed=3, spd=True)
    r = np.random.default_rng(9).standard_normal(A.n_rows)
    z0 = orc.ILU0(A.rowptr, A.colidx, A.vals).apply(r)
    z1 = orc.ILU0(A.rowptr, A.colidx, A.vals, rb_depth=0).apply(r)
    assert np.array_equal(z0, z1)
    z3 = orc.ILU0(A.rowptr, A.colidx, A.vals, rb_depth=3).apply(r)
    assert np.max(np.abs(z3 - z0)) <= 1e-12 * np.max(np.abs(z0))


@pytest.mark.parametrize("spd", [True, False])
def test_rb_preconditioned_solvers_match_dense(orc, spd):
    A = W.suitesparse_like(2048, seed=5, spd=spd)
    T = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals, classify=True)
    rp, ci, sv = T.stored_csr()
    M = orc.ILU0(rp, ci, sv, rb_depth=4)
    b = W.rhs_ones(A)
    fn = orc.cg if spd else orc.bicgstab
    r = fn(T, b, M=M, mode=orc.MODE_STATIC)
    assert r["converged"]
    x = np.linalg.solve(W.CSR(A.n_rows, A.n_cols, rp, ci, sv).dense(), b)
    assert np.linalg.norm(r["x"] - x) / np.linalg.norm(x) < 1e-8
