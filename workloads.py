"""Seeded synthetic workloads shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no classification, tiling, SpMV, dots or
solver steps).  It only builds CSR matrices (int64 rowptr, int32 colidx with strictly
increasing columns per row, float64 values) and right-hand sides, following the input
recipes in DESIGN.md ("Inputs") / SURVEY.md 8(d):

  C1  2D 5-point Poisson, m=64                         poisson2d(64)
  C2  3D 7-point Poisson m=128, value-scaled D A D      scaled_poisson3d(128, seed=1)
  C3  2D convection-diffusion m=2048, quadrant gammas   convdiff2d(2048)
  C4  SuiteSparse-shaped random, n=2^20, ~29 nnz/row    suitesparse_like(2**20, seed=42, spd=...)
  C5  3D 7-point Poisson m=512                          poisson3d(512)

b = A*1 is formed by ``rhs_ones`` as a per-row left-to-right binary64 sum
in ascending column order; x0 = 0.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class CSR:
    n_rows: int
    n_cols: int
    rowptr: np.ndarray   # int64 [n_rows+1]
    colidx: np.ndarray   # int32 [nnz]
    vals: np.ndarray     # float64 [nnz]

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])

    def dense(self) -> np.ndarray:
        d = np.zeros((self.n_rows, self.n_cols))
        rows = np.repeat(np.arange(self.n_rows), np.diff(self.rowptr))
        d[rows, self.colidx] = self.vals
        return d


def _assemble(n: int, offsets, masks, values) -> CSR:
    """Rows i get entry (i+off) with value values[k][i] where masks[k][i]; offsets ascending."""
    lens = np.zeros(n, np.int64)
    for m in masks:
        lens += m
    rowptr = np.zeros(n + 1, np.int64)
    np.cumsum(lens, out=rowptr[1:])
    nnz = int(rowptr[-1])
    colidx = np.empty(nnz, np.int32)
    vals = np.empty(nnz, np.float64)
    pos = rowptr[:-1].copy()
    idx = np.arange(n, dtype=np.int64)
    for off, m, v in zip(offsets, masks, values):
        sel = idx[m]
        p = pos[m]
        colidx[p] = (sel + off).astype(np.int32)
        vals[p] = v[m] if isinstance(v, np.ndarray) else v
        pos[m] += 1
    return CSR(n, n, rowptr, colidx, vals)


def poisson2d(m: int) -> CSR:
    """5-point Dirichlet Laplacian on an m x m grid, natural order, diag 4, off-diagonals -1."""
    n = m * m
    i = np.arange(n, dtype=np.int64)
    ix, iy = i % m, i // m
    offs = [-m, -1, 0, 1, m]
    masks = [iy > 0, ix > 0, np.ones(n, bool), ix < m - 1, iy < m - 1]
    vals = [-1.0, -1.0, 4.0, -1.0, -1.0]
    return _assemble(n, offs, masks, vals)


def poisson3d(m: int) -> CSR:
    """7-point Dirichlet Laplacian on an m^3 grid, natural order, diag 6, off-diagonals -1."""
    n = m * m * m
    i = np.arange(n, dtype=np.int64)
    ix, iy, iz = i % m, (i // m) % m, i // (m * m)
    offs = [-m * m, -m, -1, 0, 1, m, m * m]
    masks = [iz > 0, iy > 0, ix > 0, np.ones(n, bool), ix < m - 1, iy < m - 1, iz < m - 1]
    vals = [-1.0, -1.0, -1.0, 6.0, -1.0, -1.0, -1.0]
    return _assemble(n, offs, masks, vals)


def poisson3d_rows(m: int, r0: int, r1: int) -> CSR:
    """Rows [r0, r1) of poisson3d(m) with GLOBAL column ids (a rank's slab, generated without the
    rest of the matrix): the same entries in the same order as poisson3d(m) restricted to them."""
    n = m * m * m
    i = np.arange(r0, r1, dtype=np.int64)
    ix, iy, iz = i % m, (i // m) % m, i // (m * m)
    offs = [-m * m, -m, -1, 0, 1, m, m * m]
    masks = [iz > 0, iy > 0, ix > 0, np.ones(i.size, bool), ix < m - 1, iy < m - 1, iz < m - 1]
    vals = [-1.0, -1.0, -1.0, 6.0, -1.0, -1.0, -1.0]
    A = _assemble(i.size, offs, masks, vals)
    A.colidx = (A.colidx.astype(np.int64) + r0).astype(np.int32)
    A.n_cols = n
    return A


def segment_scales(n: int, seed: int = 1, seg: int = 16) -> np.ndarray:
    """d_J per 16-row segment J: 1 (p=.55), 1+2^-4 (.20), 1+2^-10 (.15), 1+u*2^-3 (.10)."""
    rng = np.random.default_rng(seed)
    nseg = (n + seg - 1) // seg
    kind = rng.choice(4, size=nseg, p=[0.55, 0.20, 0.15, 0.10])
    u = rng.random(nseg)
    d = np.where(kind == 0, 1.0, np.where(kind == 1, 1.0 + 2.0 ** -4,
                 np.where(kind == 2, 1.0 + 2.0 ** -10, 1.0 + u * 2.0 ** -3)))
    return np.repeat(d, seg)[:n]


def scaled_poisson3d(m: int, seed: int = 1) -> CSR:
    """C2: A' = D A D with A the 7-point Poisson matrix and D constant over 16-row segments.

    a'_ij = (d_i * a_ij) * d_j in binary64.  D A D stays SPD; the tiles then carry a mix of
    FP64/FP32/FP16/FP8 values."""
    A = poisson3d(m)
    d = segment_scales(A.n_rows, seed)
    rows = np.repeat(np.arange(A.n_rows), np.diff(A.rowptr))
    A.vals = (d[rows] * A.vals) * d[A.colidx]
    return A


def convdiff2d(m: int) -> CSR:
    """C3: 2D convection-diffusion, central differences scaled by h^2, Dirichlet, diag 4.

    W/E = -1 -/+ gx, S/N = -1 -/+ gy with quadrant-wise (gx, gy) chosen by the row's grid point:
      (x<1/2, y<1/2): (0, 0)                      -> FP8-exact tiles
      (x>=1/2, y<1/2): (2^-10, 2^-10)              -> FP16
      (x<1/2, y>=1/2): (2^-10+2^-20, 2^-11+2^-21)  -> FP32
      (x>=1/2, y>=1/2): (0.001, 0.0005)            -> FP64"""
    n = m * m
    i = np.arange(n, dtype=np.int64)
    ix, iy = i % m, i // m
    right, top = ix >= m // 2, iy >= m // 2
    gx = np.select([~right & ~top, right & ~top, ~right & top], [0.0, 2.0 ** -10, 2.0 ** -10 + 2.0 ** -20], 0.001)
    gy = np.select([~right & ~top, right & ~top, ~right & top], [0.0, 2.0 ** -10, 2.0 ** -11 + 2.0 ** -21], 0.0005)
    offs = [-m, -1, 0, 1, m]
    masks = [iy > 0, ix > 0, np.ones(n, bool), ix < m - 1, iy < m - 1]
    vals = [-1.0 - gy, -1.0 - gx, np.full(n, 4.0), -1.0 + gx, -1.0 + gy]
    return _assemble(n, offs, masks, vals)


def _splitmix(x: np.ndarray) -> np.ndarray:
    """64-bit splitmix hash -> uniform [0,1) (deterministic region classes)."""
    z = (x.astype(np.uint64) + np.uint64(0x9E3779B97F4A7C15))
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    z = z ^ (z >> np.uint64(31))
    return (z >> np.uint64(11)).astype(np.float64) / float(1 << 53)


def suitesparse_like(n: int = 1 << 20, seed: int = 42, spd: bool = True, per_row: int = 15) -> CSR:
    """C4: random sparse matrix shaped like SuiteSparse FEM/circuit matrices.

    Per row 15 offsets: 85% +-U{1..64}, 12% +-U{65..4096}, 3% uniform column; the pattern is
    symmetrised.  Value class per 64x64 region: 35% FP8 set {+-1,.5,.25,1.5,.75,2,3}, 25% FP16,
    20% FP32, 20% FP64 (magnitudes U[.5,2)).  Diagonal = power of two >= sum|a_ij| + 1.
    spd=True: symmetric values (SPD); spd=False: independent a_ij / a_ji and a random-sign
    diagonal (strictly diagonally dominant, so ILU(0) exists)."""
    rng = np.random.default_rng(seed)
    rows = np.repeat(np.arange(n, dtype=np.int64), per_row)
    kind = rng.choice(3, size=rows.size, p=[0.85, 0.12, 0.03])
    sign = np.where(rng.random(rows.size) < 0.5, -1, 1)
    near = rng.integers(1, 65, size=rows.size)
    far = rng.integers(65, 4097, size=rows.size)
    uni = rng.integers(0, n, size=rows.size)
    cols = np.where(kind == 0, rows + sign * near, np.where(kind == 1, rows + sign * far, uni))
    ok = (cols >= 0) & (cols < n) & (cols != rows)
    r, c = rows[ok], cols[ok]
    # symmetrise the pattern and deduplicate
    key = np.unique(np.concatenate([r * n + c, c * n + r]))
    r, c = key // n, key % n
    m = r.size

    def draw_values(count, bi, bj, gen):
        u = _splitmix(bi * np.int64(1 << 20) + bj)
        mag = gen.uniform(0.5, 2.0, size=count)
        fp8set = np.array([1.0, 0.5, 0.25, 1.5, 0.75, 2.0, 3.0])
        v = np.where(u < 0.35, fp8set[gen.integers(0, 7, size=count)],
            np.where(u < 0.60, mag.astype(np.float16).astype(np.float64),
            np.where(u < 0.80, mag.astype(np.float32).astype(np.float64), mag)))
        return v * np.where(gen.random(count) < 0.5, -1.0, 1.0)

    if spd:
        upper = r < c
        ru, cu = r[upper], c[upper]
        vu = draw_values(ru.size, ru // 64, cu // 64, rng)
        # mirror: value of (c, r) equals value of (r, c)
        rr = np.concatenate([ru, cu])
        cc = np.concatenate([cu, ru])
        vv = np.concatenate([vu, vu])
    else:
        rr, cc = r, c
        vv = draw_values(m, r // 64, c // 64, rng)
    # diagonal: power of two >= sum_j |a_ij| + 1
    rowsum = np.bincount(rr, weights=np.abs(vv), minlength=n)
    diag = np.exp2(np.ceil(np.log2(rowsum + 1.0)))
    if not spd:
        diag = diag * np.where(rng.random(n) < 0.5, -1.0, 1.0)
    rr = np.concatenate([rr, np.arange(n, dtype=np.int64)])
    cc = np.concatenate([cc, np.arange(n, dtype=np.int64)])
    vv = np.concatenate([vv, diag])
    order = np.lexsort((cc, rr))
    rr, cc, vv = rr[order], cc[order], vv[order]
    rowptr = np.zeros(n + 1, np.int64)
    np.cumsum(np.bincount(rr, minlength=n), out=rowptr[1:])
    return CSR(n, n, rowptr, cc.astype(np.int32), vv)


def rhs_ones(A: CSR) -> np.ndarray:
    """b = A * 1 as a per-row left-to-right binary64 sum in ascending column order."""
    lens = np.diff(A.rowptr)
    start = A.rowptr[:-1]
    b = np.zeros(A.n_rows)
    for k in range(int(lens.max()) if lens.size else 0):
        m = lens > k
        b[m] = b[m] + A.vals[start[m] + k]
    return b


def random_csr(n_rows: int, n_cols: int, density: float, seed: int, values: str = "mixed",
               diag: float | None = None) -> CSR:
    """Small random CSR for parity / fuzz tests.  values: 'mixed' (every precision class),
    'int' (small integers), 'f64' (uniform binary64)."""
    rng = np.random.default_rng(seed)
    mask = rng.random((n_rows, n_cols)) < density
    if diag is not None:
        np.fill_diagonal(mask, True)
    rows, cols = np.nonzero(mask)
    k = rows.size
    if values == "int":
        v = rng.integers(-4, 5, size=k).astype(np.float64)
    elif values == "f64":
        v = rng.uniform(-2, 2, size=k)
    else:
        base = rng.uniform(0.5, 2.0, size=k) * np.where(rng.random(k) < 0.5, -1, 1)
        cls = rng.integers(0, 4, size=k)
        v = np.where(cls == 0, base, np.where(cls == 1, base.astype(np.float32).astype(np.float64),
            np.where(cls == 2, base.astype(np.float16).astype(np.float64), np.round(base * 4) / 4)))
    if diag is not None:
        d = rows == cols
        v[d] = diag
    rowptr = np.zeros(n_rows + 1, np.int64)
    np.cumsum(np.bincount(rows, minlength=n_rows), out=rowptr[1:])
    return CSR(n_rows, n_cols, rowptr, cols.astype(np.int32), v)


# --------------------------------------------------------------------------- configs
CONFIGS = {
    "C1": dict(desc="CG on 2D 5-point Poisson 64x64 (n=4096), rel-residual 1e-10, 1 GPU",
               solver="cg", max_iter=1000),
    "C2": dict(desc="CG mixed precision on 3D 7-point Poisson 128^3 (2.1M rows) value-scaled tiles, 1 GPU",
               solver="cg", max_iter=1000),
    # C3: with the paper's eps = tol the dynamic switch stalls BiCGSTAB on this matrix
    # (20000 iterations, relres 6e3); eps = 1e-11 .. 1e-14 stall too, 1e-15 converges in 8455
    # iterations (FP64: 6444).  Sweep: profiles/r02_c3_eps_sweep.log (tools/c3_modes.py).
    "C3": dict(desc="BiCGSTAB on 2D convection-diffusion 2048^2 (4.2M rows), 1 GPU",
               solver="bicgstab", max_iter=20000, switch_eps=1e-15),
    "C4spd": dict(desc="PCG (ILU0) on SuiteSparse-shaped SPD, 1M rows ~29 nnz/row, 1 GPU",
                  solver="pcg", max_iter=1000),
    "C4ind": dict(desc="PBiCGSTAB (ILU0) on SuiteSparse-shaped indefinite, 1M rows, 1 GPU",
                  solver="pbicgstab", max_iter=1000),
    "C5": dict(desc="CG on 3D 7-point Poisson 512^3 (134M rows), row-partitioned",
               solver="cg", max_iter=5000),
}


def make(name: str, scale: int | None = None) -> CSR:
    """Matrix of config `name`; `scale` overrides the grid size (parity tests use small scales)."""
    if name == "C1":
        return poisson2d(scale or 64)
    if name == "C2":
        return scaled_poisson3d(scale or 128, seed=1)
    if name == "C3":
        return convdiff2d(scale or 2048)
    if name == "C4spd":
        return suitesparse_like(scale or (1 << 20), seed=42, spd=True)
    if name == "C4ind":
        return suitesparse_like(scale or (1 << 20), seed=42, spd=False)
    if name == "C5":
        return poisson3d(scale or 512)
    raise KeyError(name)
