"""Pins for the CPU baseline (oracle.baseline_solve): the OpenMP CSR
CG / BiCGSTAB / PCG / PBiCGSTAB are the textbook methods, so on FP64 tiles they must reach the
same iteration counts as the sequential oracle (Alg. 1-2, kernel order aside) and the same
solution within the stopping tolerance, with 1 and several threads."""
import numpy as np
import pytest

import workloads as W


@pytest.mark.parametrize("threads", [1, 4])
@pytest.mark.parametrize("name,kind,pre", [("C1", "cg", False), ("C3", "bicgstab", False),
                                           ("C4spd", "cg", True), ("C4ind", "bicgstab", True)])
def test_baseline_matches_oracle_fp64(orc, name, kind, pre, threads):
    A = W.make(name, {"C1": 32, "C3": 48}.get(name, 1 << 11))
    b = W.rhs_ones(A)
    T = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals, classify=False)
    M = orc.ILU0(A.rowptr, A.colidx, A.vals) if pre else None
    fn = orc.cg if kind == "cg" else orc.bicgstab
    ro = fn(T, b, M=M, mode=orc.MODE_FP64, max_iter=3000)
    rb = orc.baseline_solve(kind, A.rowptr, A.colidx, A.vals, b, M=M, max_iter=3000, threads=threads)
    assert ro["converged"] and rb["converged"] and rb["status"] == 0
    # BiCGSTAB histories move with the summation order (SURVEY c-7: up to ~9%); CG barely
    slack = ro["iterations"] // 10 if kind == "bicgstab" else ro["iterations"] // 50
    assert abs(rb["iterations"] - ro["iterations"]) <= max(2, slack)
    assert np.linalg.norm(rb["x"] - ro["x"]) / np.linalg.norm(ro["x"]) < 1e-7
    assert orc.true_relres(A.rowptr, A.colidx, A.vals, b, rb["x"]) < 1e-9
    assert rb["threads"] == threads


def test_baseline_cg_closed_form(orc):
    """CG on diag(1..k) with k distinct eigenvalues converges in k steps (finite termination)."""
    n, k = 400, 5
    d = np.repeat(np.arange(1.0, k + 1), n // k)
    A = W.CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32), d)
    r = orc.baseline_solve("cg", A.rowptr, A.colidx, A.vals, np.ones(n), tol=1e-12, threads=3)
    assert r["converged"] and r["iterations"] <= k
    assert np.allclose(r["x"], 1.0 / d, rtol=1e-12)
