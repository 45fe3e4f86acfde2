"""Pins for the oracle's rounding and the per-nonzero precision criterion.

Independent references: numpy's hardware float64->float32 cast, numpy float16 decoding,
torch's float8_e4m3fn decoding, the RNE midpoint characterisation, and the closed-form
classification table in tests/golden/classify_vectors.json.
"""
import json
import math
import os

import numpy as np
import pytest

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _e4m3_table():
    torch = pytest.importorskip("torch")
    bits = torch.arange(256, dtype=torch.int32).to(torch.uint8)
    return bits.view(torch.float8_e4m3fn).to(torch.float64).numpy()


def test_classify_golden_vectors(orc):
    g = json.load(open(os.path.join(GOLDEN, "classify_vectors.json")))
    for expr, code, why in g["vectors"]:
        v = float(eval(expr))
        assert orc.classify(v) == code, (expr, why)


def test_rne_fp32_matches_hardware_cast(orc):
    rng = np.random.default_rng(0)
    mant = rng.uniform(1, 2, 4000)
    exps = rng.integers(-160, 130, 4000)
    vals = mant * np.exp2(exps.astype(float)) * np.where(rng.random(4000) < .5, -1, 1)
    vals = np.concatenate([vals, [3.4028235677973366e38, 3.4028236e38, 1e39, 2.0 ** -149, 2.0 ** -150,
                                  1.5 * 2.0 ** -150, 2.0 ** -151]])
    with np.errstate(over="ignore"):
        ref = vals.astype(np.float32).astype(np.float64)
    got = np.array([orc.rne(v, orc.FP32) for v in vals])
    assert np.array_equal(got, ref)


def _finite_sorted_positive(table):
    v = table[np.isfinite(table) & (table >= 0)]
    return np.unique(v)


@pytest.mark.parametrize("fmt", ["fp16", "e4m3"])
def test_rne_midpoints_and_grid(orc, fmt):
    """Exhaustive characterisation of round-to-nearest-even on every binade of the format:
    grid points map to themselves, midpoints go to the even neighbour, neighbours of the
    midpoint go to the nearer grid point; beyond max: inf (FP16) / saturate 448 (E4M3)."""
    if fmt == "fp16":
        table = np.arange(65536, dtype=np.uint32).astype(np.uint16).view(np.float16).astype(np.float64)
        prec, bits_of = orc.FP16, orc.fp16_bits
    else:
        table = _e4m3_table()
        prec, bits_of = orc.FP8, orc.e4m3_bits
    grid = _finite_sorted_positive(table)
    for v in grid:
        assert orc.rne(v, prec) == v and orc.rne(-v, prec) == -v
    for a, b in zip(grid[:-1], grid[1:]):
        m = (a + b) / 2.0
        even = a if bits_of(a) % 2 == 0 else b
        assert orc.rne(m, prec) == even
        assert orc.rne(-m, prec) == -even
        assert orc.rne(np.nextafter(m, -np.inf), prec) == a
        assert orc.rne(np.nextafter(m, np.inf), prec) == b
    top = grid[-1]
    ulp = top - grid[-2]
    if fmt == "fp16":
        assert orc.rne(top + ulp / 2, prec) == np.inf          # 65520 -> inf (tie to even 2^16)
        assert orc.rne(np.nextafter(top + ulp / 2, 0), prec) == top
        assert orc.rne(1e30, prec) == np.inf
    else:
        assert orc.rne(480.0, prec) == 448.0 and orc.rne(1e30, prec) == 448.0
        assert orc.rne(-1e30, prec) == -448.0


@pytest.mark.parametrize("fmt", ["fp16", "e4m3"])
def test_bit_encodings_roundtrip(orc, fmt):
    if fmt == "fp16":
        table = np.arange(65536, dtype=np.uint32).astype(np.uint16).view(np.float16).astype(np.float64)
        enc, dec, n = orc.fp16_bits, orc.fp16_value, 65536
    else:
        table = _e4m3_table()
        enc, dec, n = orc.e4m3_bits, orc.e4m3_value, 256
    for b in range(n):
        v = table[b]
        if np.isnan(v):
            continue
        assert dec(b) == v or (v == 0 and dec(b) == 0)
        assert enc(v) == b


def test_every_representable_value_classifies_at_or_below_its_format(orc):
    """Each decoded E4M3 value classifies FP8; each FP16 value classifies FP16 or FP8."""
    for v in _finite_sorted_positive(_e4m3_table()):
        assert orc.classify(v) == orc.FP8 and orc.classify(-v) == orc.FP8
    fp16 = np.arange(65536, dtype=np.uint32).astype(np.uint16).view(np.float16).astype(np.float64)
    for v in fp16[np.isfinite(fp16)][::7]:
        assert orc.classify(v) in (orc.FP16, orc.FP8)


def test_classification_boundary_is_relative(orc):
    # the loss criterion is relative (reading R1): scaling by a power of two keeps the class
    for v in [1 + 2 ** -50, 1 + 2 ** -10, 1 + 2 ** -23, 0.1]:
        c = orc.classify(v)
        assert orc.classify(v * 2.0 ** -3) == c
    assert math.isclose(abs((1 + 2 ** -49) - orc.rne(1 + 2 ** -49, orc.FP32)), 2 ** -49)
