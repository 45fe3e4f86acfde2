"""Pins for the oracle's CSR -> two-level tile converter (Fig. 5;
canonical form DESIGN.md "Canonical tile format").

Each check rebuilds the matrix from the canonical arrays with code written here, independent
of the converter: dense round trip, brute force over tile patterns, Fig. 6 structure.
"""
import itertools
import json
import os

import numpy as np
import pytest

import workloads as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _decode_table_e4m3():
    torch = pytest.importorskip("torch")
    bits = torch.arange(256, dtype=torch.int32).to(torch.uint8)
    return bits.view(torch.float8_e4m3fn).to(torch.float64).numpy()


E4M3 = None


def stored_value(arr, t, a):
    global E4M3
    p, o = arr["TilePrec"][t], arr["ValOff"][t] + a
    if p == 0:
        return arr["Val64"][o]
    if p == 1:
        return float(arr["Val32"][o])
    if p == 2:
        return float(arr["Val16"][o:o + 1].view(np.float16)[0])
    if E4M3 is None:
        E4M3 = _decode_table_e4m3()
    return E4M3[arr["Val8"][o]]


def dense_from_tiles(arr, n_rows, n_cols, T):
    D = np.zeros((n_rows, n_cols))
    P = np.zeros((n_rows, n_cols), bool)
    nt = len(arr["TileRowidx"])
    for t in range(nt):
        tr, tc = arr["TileRowidx"][t], arr["TileColidx"][t]
        r0, r1 = arr["Nonrow"][t], arr["Nonrow"][t + 1]
        tile_nnz = arr["TileNnz"][t + 1] - arr["TileNnz"][t]
        assert r1 > r0, "tiles are non-empty"
        prev_lr = -1
        for ri in range(r0, r1):
            lr = arr["RowIndex"][ri]
            assert lr > prev_lr and lr < T
            prev_lr = lr
            s = arr["CsrRowptr"][ri]
            e = arr["CsrRowptr"][ri + 1] if ri + 1 < r1 else tile_nnz
            assert e > s
            prev_lc = -1
            for a in range(s, e):
                lc = arr["CsrColidx"][arr["TileNnz"][t] + a]
                assert lc > prev_lc and lc < T
                prev_lc = lc
                i, j = tr * T + lr, tc * T + lc
                assert not P[i, j]
                P[i, j] = True
                D[i, j] = stored_value(arr, t, a)
    return D, P


def check_structure(arr, A, T):
    keys = arr["TileRowidx"].astype(np.int64) * (10 ** 9) + arr["TileColidx"]
    assert np.all(np.diff(keys) > 0), "tiles sorted by (row, col), distinct"
    assert arr["TileNnz"][0] == 0 and arr["TileNnz"][-1] == A.nnz
    assert arr["Nonrow"][0] == 0 and arr["Nonrow"][-1] == len(arr["RowIndex"])
    ntr = (A.n_rows + T - 1) // T
    trp = arr["TileRowPtr"]
    assert len(trp) == ntr + 1 and trp[-1] == len(keys)
    for TR in range(ntr):
        assert np.all(arr["TileRowidx"][trp[TR]:trp[TR + 1]] == TR)
    # typed arrays: each tile's values contiguous in its precision's array, tiles in order
    for p, name in enumerate(["Val64", "Val32", "Val16", "Val8"]):
        sel = np.nonzero(arr["TilePrec"] == p)[0]
        expect = 0
        for t in sel:
            assert arr["ValOff"][t] == expect
            expect += arr["TileNnz"][t + 1] - arr["TileNnz"][t]
        assert expect == len(arr[name])


def roundtrip(orc, A, T, classify=True):
    tiles = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals, T=T, classify=classify)
    arr = tiles.arrays()
    check_structure(arr, A, T)
    D, P = dense_from_tiles(arr, A.n_rows, A.n_cols, T)
    ref = A.dense()
    refP = np.zeros_like(P)
    rows = np.repeat(np.arange(A.n_rows), np.diff(A.rowptr))
    refP[rows, A.colidx] = True
    assert np.array_equal(P, refP), "pattern preserved (explicit zeros kept)"
    if not classify:
        assert np.array_equal(D, ref)
        assert np.all(arr["TilePrec"] == 0)
    else:
        # criterion: every stored value within 1e-15 relative of its original
        assert np.all(np.abs(D - ref) < 1e-15 * np.abs(ref) + (ref == 0))
    return tiles, arr


@pytest.mark.parametrize("T", [2, 3, 16])
@pytest.mark.parametrize("seed", range(4))
def test_random_roundtrip(orc, T, seed):
    A = W.random_csr(37, 41, 0.15, seed, values="mixed")
    roundtrip(orc, A, T)
    roundtrip(orc, A, T, classify=False)


def test_tileprec_is_minimal_and_floor(orc):
    """TilePrec = the highest precision any nonzero needs: lowering it one step would break the
    criterion for some nonzero; floor_t never exceeds TilePrec and holds the normal range."""
    A = W.random_csr(64, 64, 0.2, 7, values="mixed")
    A.vals[::11] *= 1e-3            # some small magnitudes to exercise the range floor
    tiles, arr = roundtrip(orc, A, 16)
    rp, ci, v = A.rowptr, A.colidx, A.vals
    for t in range(tiles.tilenum):
        p = arr["TilePrec"][t]
        assert arr["Floor"][t] >= p
        tr, tc = arr["TileRowidx"][t], arr["TileColidx"][t]
        vals = [v[k] for i in range(tr * 16, tr * 16 + 16) for k in range(rp[i], rp[i + 1]) if ci[k] // 16 == tc]
        if p < 3:
            lower = p + 1
            assert any(abs(x - orc.rne(x, lower)) >= 1e-15 * abs(x) for x in vals if x != 0)
        lo = {1: 2.0 ** -126, 2: 2.0 ** -14, 3: 2.0 ** -6}
        hi = {1: 3.4028234663852886e38, 2: 65504.0, 3: 448.0}
        f = arr["Floor"][t]
        stored = [stored_value(arr, t, a) for a in range(arr["TileNnz"][t + 1] - arr["TileNnz"][t])]
        if f > p:
            assert all(s == 0 or lo[f] <= abs(s) <= hi[f] for s in stored)
        if f < 3:
            g = f + 1
            assert not all(s == 0 or lo[g] <= abs(s) <= hi[g] for s in stored)


def test_bruteforce_all_patterns_4x4_T2(orc):
    """Every sparsity pattern of a 4x4 matrix (2x2 grid of 2x2 tiles): 65536 patterns."""
    n = 4
    for mask in range(1 << 16):
        bits = [(mask >> b) & 1 for b in range(16)]
        rows, cols = np.nonzero(np.array(bits).reshape(4, 4))
        rowptr = np.zeros(n + 1, np.int64)
        np.cumsum(np.bincount(rows, minlength=n), out=rowptr[1:])
        vals = np.arange(1, len(rows) + 1, dtype=np.float64)
        A = W.CSR(n, n, rowptr, cols.astype(np.int32), vals)
        tiles = orc.Tiles(n, n, rowptr, cols, vals, T=2)
        arr = tiles.arrays()
        D, P = dense_from_tiles(arr, n, n, 2)
        assert np.array_equal(D, A.dense())
        expect_tiles = len({(r // 2, c // 2) for r, c in zip(rows, cols)})
        assert tiles.tilenum == expect_tiles


def test_bruteforce_all_tile_patterns_T3(orc):
    """Every pattern of one 3x3 tile, placed at each of the four tile positions of a 6x6
    matrix (plus a fixed diagonal elsewhere) with T = 3."""
    n = 6
    for mask in range(1, 1 << 9):
        tp = np.array([(mask >> b) & 1 for b in range(9)]).reshape(3, 3)
        for (bi, bj) in itertools.product(range(2), range(2)):
            M = np.eye(n, dtype=bool)
            M[bi * 3:bi * 3 + 3, bj * 3:bj * 3 + 3] |= tp.astype(bool)
            rows, cols = np.nonzero(M)
            rowptr = np.zeros(n + 1, np.int64)
            np.cumsum(np.bincount(rows, minlength=n), out=rowptr[1:])
            vals = (np.arange(len(rows)) % 7 + 0.5).astype(np.float64)
            A = W.CSR(n, n, rowptr, cols.astype(np.int32), vals)
            tiles = orc.Tiles(n, n, rowptr, cols, vals, T=3)
            arr = tiles.arrays()
            D, _ = dense_from_tiles(arr, n, n, 3)
            assert np.array_equal(D, A.dense())


def test_fig6_structure(orc):
    """Fig. 6: 6x6, 2x2 tiles, five tiles in three row tiles with d_s = [1,2,2]
    tiles per row tile and three vector segments."""
    g = json.load(open(os.path.join(GOLDEN, "fig6.json")))
    # a 6x6 pattern with tiles (0,0); (1,0),(1,1); (2,1),(2,2)  (the image is missing)
    pat = {(0, 0), (0, 1), (1, 1), (2, 0), (2, 2), (3, 3), (4, 3), (4, 4), (5, 5)}
    rows = np.array(sorted(pat))
    rowptr = np.zeros(7, np.int64)
    np.cumsum(np.bincount(rows[:, 0], minlength=6), out=rowptr[1:])
    tiles = orc.Tiles(6, 6, rowptr, rows[:, 1], np.full(len(rows), 2.0), T=g["T"])
    arr = tiles.arrays()
    assert tiles.tilenum == g["tilenum"]
    assert list(np.diff(arr["TileRowPtr"])) == g["d_s"]
    assert (g["n"] + g["T"] - 1) // g["T"] == g["n_segments"]


@pytest.mark.parametrize("name,scale,tiles,rownum", [("C1", 64, 1144, 12544), ("C3", 2048, 1306368, 13099008)])
def test_config_tile_counts_match_closed_form(orc, name, scale, tiles, rownum):
    """Tile and non-empty-row counts of the stencil configs (closed form)."""
    if scale > 1000:
        pytest.skip("full-size C3 conversion is covered by the slow suite")
    A = W.make(name, scale)
    t = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
    assert (t.tilenum, t.rownum) == (tiles, rownum)


def test_poisson3d_tile_closed_form(orc):
    """3D m^3 Poisson with S = m/16: tiles = m^2 S + m^2 (2S-2) + 2 m S (2m-2)."""
    for m in (16, 32):
        A = W.poisson3d(m)
        S = m // 16
        t = orc.Tiles(A.n_rows, A.n_cols, A.rowptr, A.colidx, A.vals)
        assert t.tilenum == m * m * S + m * m * (2 * S - 2) + 2 * m * S * (2 * m - 2)
        assert t.rownum == 16 * m * m * S + m * m * (2 * S - 2) + 32 * m * S * (2 * m - 2)


def test_invalid_inputs(orc):
    rp = np.array([0, 2, 3], np.int64)
    assert orc.csr_validate(2, 2, rp, np.array([1, 0, 1], np.int32), np.ones(3)) == orc.ERR_UNSORTED_CSR
    assert orc.csr_validate(2, 2, rp, np.array([0, 0, 1], np.int32), np.ones(3)) == orc.ERR_UNSORTED_CSR
    assert orc.csr_validate(2, 2, rp, np.array([0, 1, 1], np.int32), np.array([1, np.nan, 1])) == orc.ERR_NONFINITE
    assert orc.csr_validate(2, 2, rp, np.array([0, 2, 1], np.int32), np.ones(3)) == orc.ERR_INVALID_ARG
    assert orc.csr_validate(2, 2, np.array([0, 3, 2], np.int64), np.array([0, 1, 1], np.int32), np.ones(3)) \
        == orc.ERR_INVALID_ARG
    with pytest.raises(orc.OracleError):
        orc.Tiles(2, 2, rp, np.array([1, 0, 1], np.int32), np.ones(3))


def test_empty_and_ragged(orc):
    """An all-empty matrix; empty rows inside tile rows; n not a multiple of T."""
    A = W.CSR(5, 5, np.zeros(6, np.int64), np.zeros(0, np.int32), np.zeros(0))
    t = orc.Tiles(5, 5, A.rowptr, A.colidx, A.vals)
    assert t.tilenum == 0 and t.rownum == 0
    C = W.random_csr(35, 35, 0.1, 3, values="f64")
    rows = np.repeat(np.arange(35), np.diff(C.rowptr))
    m = (rows < 10) | (rows >= 19)              # rows 10..18 empty
    rowptr = np.zeros(36, np.int64)
    np.cumsum(np.bincount(rows[m], minlength=35), out=rowptr[1:])
    roundtrip(orc, W.CSR(35, 35, rowptr, C.colidx[m], C.vals[m]), 16)
