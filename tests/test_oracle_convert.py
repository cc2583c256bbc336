"""Pins for the oracle's software converter.

Each pin is independent of oracle.c's arithmetic: x86 hardware converters
(F16C, AVX512-FP16, SSE2 cvtsd2ss), numpy's converters, and the paper's
fixed points (tests/golden/convert_fixed_points.txt).
"""
import os
import subprocess

import numpy as np
import pytest

import oracle

HERE = os.path.dirname(os.path.abspath(__file__))
CODE = {"f64": 0, "f32": 1, "f16": 2}


def _hw(hwcheck, mode, count=None):
    args = [hwcheck, mode] + ([str(count)] if count else [])
    out = subprocess.run(args, capture_output=True, text=True)
    line = out.stdout.strip()
    if line.startswith("skip="):
        pytest.skip(line)
    assert out.returncode == 0, line + out.stderr
    assert "mismatches=0" in line, line


def test_fixed_points_golden(oracle_lib):
    n = 0
    for raw in open(os.path.join(HERE, "golden", "convert_fixed_points.txt")):
        fields = raw.split("#")[0].split()
        if not fields:
            continue
        s, d, x, e = fields
        got = oracle.convert_bits(int(x, 16), CODE[s], CODE[d])
        assert got == int(e, 16), (raw, hex(got))
        n += 1
    assert n >= 40


def test_f32_to_f16_all_2pow32_vs_f16c(hwcheck):
    """All 2^32 fp32 bit patterns vs x86 F16C vcvtps2ph (RNE)."""
    _hw(hwcheck, "f32f16")


def test_f16_widening_all_2pow16_vs_f16c(hwcheck):
    _hw(hwcheck, "f16wide")


def test_f64_to_f16_vs_avx512fp16(hwcheck):
    """Every fp16 midpoint +-4 fp64 ulps, plus 2^25 random patterns, vs vcvtsd2sh."""
    _hw(hwcheck, "f64f16", 1 << 25)


def test_f64_to_f32_vs_sse(hwcheck):
    _hw(hwcheck, "f64f32", 1 << 24)


def test_f32_to_f64_exact(hwcheck):
    _hw(hwcheck, "f32f64", 1 << 24)


def _nan_aware_equal(a_bits, b_bits, a_nan):
    eq = a_bits == b_bits
    return np.all(eq | a_nan)


def test_f32_to_f16_vs_numpy_sample(oracle_lib):
    rng = np.random.default_rng(1)
    bits = rng.integers(0, 2**32, size=1 << 22, dtype=np.uint64).astype(np.uint32)
    x = bits.view(np.float32)
    with np.errstate(all="ignore"):
        ref = x.astype(np.float16).view(np.uint16)
    got = oracle.convert(x, 1, 2).view(np.uint16)
    assert _nan_aware_equal(got, ref, np.isnan(x))


def test_f64_to_f16_vs_numpy_direct(oracle_lib):
    """numpy converts float64 -> float16 directly (single rounding)."""
    rng = np.random.default_rng(2)
    e = rng.integers(1023 - 30, 1023 + 18, size=1 << 20, dtype=np.uint64)
    m = rng.integers(0, 2**52, size=1 << 20, dtype=np.uint64)
    s = rng.integers(0, 2, size=1 << 20, dtype=np.uint64)
    x = ((s << np.uint64(63)) | (e << np.uint64(52)) | m).view(np.float64)
    with np.errstate(all="ignore"):
        ref = x.astype(np.float16).view(np.uint16)
    got = oracle.convert(x, 0, 2).view(np.uint16)
    assert np.array_equal(got, ref)


def test_all_f16_widen_and_round_trip(oracle_lib):
    h = np.arange(65536, dtype=np.uint32).astype(np.uint16).view(np.float16)
    nan = np.isnan(h)
    w32 = oracle.convert(h, 2, 1)
    w64 = oracle.convert(h, 2, 0)
    assert np.array_equal(w32[~nan], h[~nan].astype(np.float32))
    assert np.array_equal(w64[~nan], h[~nan].astype(np.float64))
    assert np.all(w32[nan].view(np.uint32) == 0x7FFFFFFF)
    back = oracle.convert(w32, 1, 2).view(np.uint16)
    assert np.array_equal(back[~nan], h[~nan].view(np.uint16))
    back64 = oracle.convert(w64, 0, 2).view(np.uint16)
    assert np.array_equal(back64[~nan], h[~nan].view(np.uint16))
    assert np.all(back[nan] == 0x7FFF)


def test_direct_vs_transient_differ(oracle_lib):
    """transient conversion (via an intermediate type) can add error; the
    oracle's direct f64->f16 must differ from f64->f32->f16 on the witnesses."""
    for x in [1 + 2**-11 + 2**-30, 2**-25 * (1 + 2**-30), 65520 - 2**-30]:
        b = np.array([x]).view(np.uint64)[0]
        direct = oracle.convert_bits(int(b), 0, 2)
        via = oracle.convert_bits(oracle.convert_bits(int(b), 0, 1), 1, 2)
        assert direct != via


def test_convert_identity_and_empty(oracle_lib):
    a = np.array([1.5, -2.25, 3.0], dtype=np.float32)
    assert np.array_equal(oracle.convert(a, 1, 1), a)
    assert oracle.convert(np.zeros(0, np.float32), 1, 2).size == 0
