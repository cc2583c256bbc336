"""Pins for the oracle's bf16 extension (reading #28).

bf16 = sign, 8 exponent bits (bias 127), 7 fraction bits; RNE narrowing with
subnormals and overflow to inf, canonical NaN 0x7FFF (reading #5's pattern).
Independent of oracle.c: x86 AVX512-BF16 hardware (vcvtneps2bf16, all 2^32
normal inputs), torch's CPU bfloat16 cast (f32 subnormals), and an exact
rational-arithmetic RNE written here for fp64 inputs (single rounding).
"""
import os
import subprocess
from fractions import Fraction

import numpy as np
import pytest

import oracle

F64, F32, F16, BF16 = 0, 1, 2, 3


def _hw(hwcheck, mode):
    out = subprocess.run([hwcheck, mode], capture_output=True, text=True)
    line = out.stdout.strip()
    if line.startswith("skip="):
        pytest.skip(line)
    assert out.returncode == 0 and "mismatches=0" in line, line + out.stderr


def test_f32_to_bf16_all_normal_vs_avx512bf16(hwcheck):
    _hw(hwcheck, "f32bf16")


def test_bf16_widening_all_2pow16(hwcheck):
    _hw(hwcheck, "bf16wide")


def test_f32_subnormals_to_bf16_vs_torch(oracle_lib):
    """Every f32 subnormal (both signs) vs torch's CPU bfloat16 cast (RNE)."""
    import torch
    lo = np.arange(1, 1 << 23, dtype=np.uint32)
    bits = np.concatenate([lo, lo | np.uint32(0x80000000)])
    want = torch.from_numpy(bits.view(np.float32).copy()).to(torch.bfloat16).view(torch.int16)
    want = want.numpy().view(np.uint16)
    got = oracle.convert(bits.view(np.float32), F32, BF16)
    assert np.array_equal(got, want)


def _rne_bf16_exact(x: float) -> int:
    """RNE of the exact value of fp64 x to bf16 bits, by rational arithmetic."""
    if x != x:
        return 0x7FFF
    sign = 0x8000 if (x < 0 or (x == 0 and np.signbit(x))) else 0
    if x in (float("inf"), float("-inf")):
        return sign | 0x7F80
    a = abs(Fraction(x))
    if a == 0:
        return sign
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if Fraction(2) ** e > a:
        e -= 1                                    # 2^e <= a < 2^(e+1)
    q = max(e, -126) - 7                          # quantum exponent
    k = a / Fraction(2) ** q
    K = int(k)
    rem = k - K
    if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and K % 2 == 1):
        K += 1
    if K == 0:
        return sign
    if K == 256:                                  # carry: 2^8 * 2^q = 2^7 * 2^(q+1)
        K, q = 128, q + 1
    if K >= 128:                                  # normal (8 significant bits)
        biased = q + 7 + 127
        if biased >= 255:
            return sign | 0x7F80
        return sign | (biased << 7) | (K - 128)
    return sign | K                               # subnormal (q == -133)


def _bf16_value(h: int) -> float:
    return float(np.uint32(h << 16).view(np.float32))


def test_f64_to_bf16_single_rounding_vs_exact(oracle_lib):
    """Every positive finite bf16 value and midpoint +-0..3 fp64 ulps (incl. the
    subnormal and overflow edges), both signs, plus random fp64 patterns: the
    oracle's one-step f64 -> bf16 equals the exact rational RNE."""
    pts = []
    for h in range(0, 0x7F80):
        v = _bf16_value(h)
        nxt = Fraction(_bf16_value(h + 1)) if h + 1 < 0x7F80 else Fraction(2) ** 128   # overflow edge
        mid = float((Fraction(v) + nxt) / 2)
        for base in (v, mid):
            up = dn = base
            pts.append(base)
            for _ in range(3):
                up = float(np.nextafter(up, np.inf))
                dn = float(np.nextafter(dn, -np.inf))
                pts += [up, dn]
    rng = np.random.default_rng(5)
    rnd = rng.integers(0, 1 << 63, size=20000, dtype=np.int64).view(np.float64)
    arr = np.array(pts + [-p for p in pts] + list(rnd) + [float("nan"), float("inf"), -0.0])
    got = oracle.convert(arr, F64, BF16)
    want = np.array([_rne_bf16_exact(float(x)) for x in arr], dtype=np.uint16)
    bad = np.flatnonzero(got != want)
    assert bad.size == 0, [(arr[i], hex(got[i]), hex(want[i])) for i in bad[:5]]


def test_bf16_double_rounding_witness(oracle_lib):
    """f64 -> bf16 is ONE rounding: 1 + 2^-8 + 2^-40 rounds up to 1 + 2^-7 (0x3F81),
    while rounding via f32 first would hit the tie 1 + 2^-8 and give 0x3F80."""
    x = 1.0 + 2.0 ** -8 + 2.0 ** -40
    assert oracle.convert_bits(np.float64(x).view(np.uint64).item(), F64, BF16) == 0x3F81
    via = oracle.convert_bits(oracle.convert_bits(np.float64(x).view(np.uint64).item(), F64, F32), F32, BF16)
    assert via == 0x3F80


def test_radix4_codec_bijection(oracle_lib):
    for m in range(1, 6):
        seen = set()
        for cid in range(4 ** m):
            p = oracle.config_decode(m, cid, 4)
            assert all(0 <= x <= 3 for x in p) and oracle.config_encode(p, 4) == cid
            seen.add(tuple(p))
        assert len(seen) == 4 ** m
    # radix 3 ids are unchanged (paper space), and bf16 is rejected there
    assert oracle.config_decode(3, 13) == [1, 1, 1]
    with pytest.raises(ValueError):
        oracle.config_encode([3, 1, 1])


# --------------------------------------------------- apps with bf16 objects
APP_DIMS = {"gemm": [13, 17, 11], "2mm": [9, 14, 11, 7], "3mm": [6, 9, 8, 10, 7],
            "atax": [300, 77], "bicg": [270, 93], "gesummv": [75], "mvt": [301],
            "syrk": [23, 14], "syr2k": [21, 13], "conv2d": [15, 21], "corr": [60, 17],
            "covar": [55, 13], "conv3d": [6, 7, 9], "fdtd2d": [3, 11, 13]}


@pytest.mark.parametrize("kind", ["gemm", "2mm", "3mm", "atax", "bicg", "gesummv", "mvt", "syrk",
                                  "syr2k"])
def test_bf16_configs_exact_integer_results(oracle_lib, kind):
    """Small non-negative integers (< 8) with every partial sum an integer: any
    radix-4 configuration whose objects hold those integers exactly (bf16: |v| <=
    256) reproduces exact integer arithmetic -- bf16 loads widen exactly, its
    stores round exactly, and the statements compute in f32 (reading #28)."""
    from test_oracle_apps import numpy_ref, _exact_ints
    rng = np.random.default_rng(17)
    dims = APP_DIMS[kind]
    objs = oracle.app_objects(kind, dims)
    ins = _exact_ints(kind, dims, objs, rng)
    sc = (2.0, 3.0) if kind in ("gemm", "gesummv", "syrk", "syr2k") else None
    if kind == "syrk":
        ins[1] = np.triu(ins[1]) + np.triu(ins[1], 1).T
    exact = {m: np.rint(v) for m, v in numpy_ref(kind, ins, objs, sc, dims).items()}
    lim = {F64: 2.0 ** 53, F32: 2.0 ** 24, F16: 2048.0, BF16: 256.0}
    ids = [c for c in range(4 ** len(objs)) if BF16 in oracle.config_decode(len(objs), c, 4)]
    ids = list(np.random.default_rng(3).permutation(ids)[:150])
    n_checked = 0
    for cid in ids:
        prec = oracle.config_decode(len(objs), int(cid), 4)
        if not all(np.all(np.abs(v) <= lim[prec[m]]) for m, v in exact.items()):
            continue
        fin = oracle.run_config(kind, dims, prec, ins, sc)
        for m, v in exact.items():
            assert np.array_equal(oracle.widen(fin[m], prec[m]).reshape(v.shape), v), (prec, m)
        n_checked += 1
    assert n_checked >= min(10, len(ids) // 3), n_checked


def test_bf16_store_is_rne_of_f32_result(oracle_lib):
    """GEMM with C in bf16 and A, B in f32: C_bf16 == RNE_bf16(C of the all-f32 run)
    (T = f32 either way; the only difference is the final store), element by element."""
    dims = [33, 29, 41]
    objs = oracle.app_objects("gemm", dims)
    from paper_conf_cgo_kangcp20_b200 import inputs as gen
    ins = gen.make_inputs("gemm", objs, "random", seed=2)
    # C is inout: its input must be the same in both runs, and exactly bf16
    ins[2] = oracle.widen(oracle.convert(ins[2], F32, BF16), BF16).astype(np.float32)
    f32 = oracle.run_config("gemm", dims, [F32, F32, F32], ins, (1.5, 1.2))
    b16 = oracle.run_config("gemm", dims, [F32, F32, BF16], ins, (1.5, 1.2))
    assert np.array_equal(b16[2], oracle.convert(f32[2], F32, BF16))


def test_bf16_quality_closed_forms(oracle_lib):
    ref = np.array([1.0, 2.0, 4.0, 3.0])
    out = oracle.convert(np.array([1.0, 2.0, 4.0, 3.0], dtype=np.float32), F32, BF16)
    assert oracle.quality(out, BF16, ref)["quality"] == 1.0
    out = oracle.convert(np.array([1.0, 2.0 * (1 + 2 ** -7), 4.0, 3.0], dtype=np.float32), F32, BF16)
    q = oracle.quality(out, BF16, ref)
    assert q["quality"] == 1.0 - (2 ** -7) / 4 and q["nonfinite"] == 0
    big = oracle.convert(np.array([3.5e38], dtype=np.float32), F32, BF16)   # > bf16 max -> inf
    assert oracle.quality(big, BF16, np.array([3.5e38]))["nonfinite"] == 1
