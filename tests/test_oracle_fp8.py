"""Pins for the oracle's fp8 object types (reading #29).

E4M3 = OCP FP8 "fn" (bias 7, 3 fraction bits, no infinity, NaN = S.1111.111,
max 448); E5M2 = IEEE-like (bias 15, 2 fraction bits, inf, max 57344).  An fp8
object carries a per-tensor power-of-two scale 2^k chosen from its amax.

Independent of oracle.c's bit-shifting converter:
  * the 256 codes of each format decoded from the OCP field definition here;
  * torch's CPU float8 casts over all 2^32 f32 inputs (NaN-ness only for NaN);
  * a brute-force nearest-value search over the finite code table with
    ties-to-even, on fp64 inputs (midpoints +- ulps, random);
  * the scale rule's defining inequality and closed forms;
  * exact-integer app invariants and an independently rounded GEMM output.
"""
from concurrent.futures import ThreadPoolExecutor

import numpy as np
import pytest

import oracle

F64, F32, F16, BF16, E4M3, E5M2 = 0, 1, 2, 3, 4, 5
FMT = {E4M3: (4, 3, 7), E5M2: (5, 2, 15)}


def _ocp_value(code: int, t: int) -> float:
    """Value of an fp8 code from the OCP field definition (not oracle.c)."""
    eb, mb, bias = FMT[t]
    s = -1.0 if code & 0x80 else 1.0
    e = (code >> mb) & ((1 << eb) - 1)
    f = code & ((1 << mb) - 1)
    if t == E4M3 and e == 15 and f == 7:
        return float("nan")
    if t == E5M2 and e == 31:
        return s * float("inf") if f == 0 else float("nan")
    if e == 0:
        return s * f * 2.0 ** (1 - bias - mb)
    return s * (1 + f / 2 ** mb) * 2.0 ** (e - bias)


@pytest.mark.parametrize("t", [E4M3, E5M2])
def test_fp8_decode_all_codes(oracle_lib, t):
    codes = np.arange(256, dtype=np.uint8)
    got = oracle.widen(codes, t)
    want = np.array([_ocp_value(c, t) for c in range(256)])
    nan = np.isnan(want)
    assert np.array_equal(np.isnan(got), nan)
    assert np.array_equal(got[~nan], want[~nan])
    # signed zeros keep their sign
    assert np.signbit(got[0x80]) and not np.signbit(got[0])


def test_fp8_fixed_points(oracle_lib):
    """OCP maxima, smallest subnormals, overflow rule, ties to even, canonical NaN."""
    f = lambda v, t: int(oracle.convert(np.array([v], np.float64), F64, t)[0])
    assert f(448.0, E4M3) == 0x7E and f(-448.0, E4M3) == 0xFE
    assert f(464.0, E4M3) == 0x7E            # tie between 448 and (480) -> even 448
    assert f(464.0 + 2 ** -40, E4M3) == 0x7F  # rounds past 448 -> NaN (no inf)
    assert f(float("inf"), E4M3) == 0x7F and f(float("-inf"), E4M3) == 0x7F
    assert f(2.0 ** -9, E4M3) == 0x01 and f(2.0 ** -10, E4M3) == 0x00   # tie -> 0
    assert f(3 * 2.0 ** -10, E4M3) == 0x02                              # tie -> even
    assert f(57344.0, E5M2) == 0x7B and f(61440.0, E5M2) == 0x7C        # tie at the edge -> inf
    assert f(61440.0 - 2 ** -30, E5M2) == 0x7B
    assert f(float("-inf"), E5M2) == 0xFC
    assert f(2.0 ** -16, E5M2) == 0x01 and f(2.0 ** -17, E5M2) == 0x00
    assert f(float("nan"), E4M3) == 0x7F and f(float("nan"), E5M2) == 0x7F
    assert f(-0.0, E4M3) == 0x80 and f(-0.0, E5M2) == 0x80
    assert f(1.0625, E4M3) == 0x38 and f(1.1875, E4M3) == 0x3A           # ties to even


def _chunk_vs_torch(args):
    import torch
    lo, hi, t = args
    bits = np.arange(lo, hi, dtype=np.uint64).astype(np.uint32)
    x = bits.view(np.float32)
    tdt = torch.float8_e4m3fn if t == E4M3 else torch.float8_e5m2
    want = torch.from_numpy(x).to(tdt).view(torch.uint8).numpy()
    got = oracle.convert(x, F32, t)
    wn = np.isnan(oracle.widen(want, t))
    gn = np.isnan(oracle.widen(got, t))
    bad = int(np.count_nonzero(wn != gn)) + int(np.count_nonzero((got != want) & ~gn))
    return bad


@pytest.mark.parametrize("t", [E4M3, E5M2])
def test_f32_to_fp8_all_2pow32_vs_torch(oracle_lib, t):
    """Every f32 bit pattern vs torch's float8 cast (RNE; E4M3 overflow -> NaN,
    E5M2 overflow -> inf); NaN codes compared by NaN-ness (reading #5 drops the sign)."""
    step = 1 << 26
    jobs = [(lo, lo + step, t) for lo in range(0, 1 << 32, step)]
    with ThreadPoolExecutor(8) as ex:
        bad = sum(ex.map(_chunk_vs_torch, jobs))
    assert bad == 0


def _nearest_fp8(v: np.ndarray, t: int) -> np.ndarray:
    """Brute force: nearest finite code value, ties to the even code (fraction
    LSB 0), beyond the overflow midpoint -> inf (E5M2) / NaN (E4M3)."""
    codes = np.arange(128, dtype=np.int64)                 # non-negative codes
    vals = np.array([_ocp_value(int(c), t) for c in codes])
    fin = np.isfinite(vals)
    codes, vals = codes[fin], vals[fin]
    order = np.argsort(vals, kind="stable")
    codes, vals = codes[order], vals[order]
    # drop the duplicate +0 ordering issue: values are strictly increasing here
    a = np.abs(v)
    hi = np.searchsorted(vals, a, side="left")
    hi = np.clip(hi, 0, len(vals) - 1)
    lo = np.clip(hi - 1, 0, len(vals) - 1)
    dlo, dhi = np.abs(a - vals[lo]), np.abs(vals[hi] - a)
    pick = np.where(dlo < dhi, lo, np.where(dhi < dlo, hi, np.where(codes[lo] % 2 == 0, lo, hi)))
    out = codes[pick].astype(np.int64)
    vmax = vals[-1]
    step_top = vals[-1] - vals[-2]
    over = a >= vmax + step_top / 2
    if t == E4M3:                                            # next value would be 480 (NaN code)
        over = (a > vmax + step_top / 2) | ((a == vmax + step_top / 2) & (codes[-1] % 2 == 1))
    out = np.where(over, 0x7C if t == E5M2 else 0x7F, out)
    sign = np.signbit(v).astype(np.int64) << 7
    out = np.where(over & (t == E4M3), 0x7F, out | sign)
    return out.astype(np.uint8)


@pytest.mark.parametrize("t", [E4M3, E5M2])
def test_f64_to_fp8_vs_brute_force(oracle_lib, t):
    """fp64 -> fp8 in one rounding vs a nearest-value search: every midpoint
    between consecutive codes +- 0..4 fp64 ulps, plus 2^20 random values."""
    vals = np.array(sorted({abs(_ocp_value(c, t)) for c in range(128)} - {float("nan")}))
    vals = vals[np.isfinite(vals)]
    mids = (vals[:-1] + vals[1:]) / 2
    mids = np.concatenate([mids, [vals[-1] + (vals[-1] - vals[-2]) / 2]])   # overflow edge
    cand = [mids]
    up, dn = mids.copy(), mids.copy()
    for _ in range(4):
        up, dn = np.nextafter(up, np.inf), np.nextafter(dn, -np.inf)
        cand += [up, dn]
    rng = np.random.default_rng(29)
    fmax = vals[-1]
    cand += [rng.uniform(0, 1.2 * fmax, 1 << 19), np.exp2(rng.uniform(-20, 17, 1 << 19)), vals]
    x = np.concatenate(cand)
    x = np.concatenate([x, -x])
    got = oracle.convert(x, F64, t)
    want = _nearest_fp8(x, t)
    if t == E4M3:                                           # NaN codes: compare NaN-ness
        gn, wn = np.isnan(oracle.widen(got, t)), np.isnan(oracle.widen(want, t))
        assert np.array_equal(gn, wn)
        assert np.array_equal(got[~gn], want[~gn])
    else:
        assert np.array_equal(got, want)


@pytest.mark.parametrize("t", [E4M3, E5M2])
def test_fp8_widening_exact_and_roundtrip(oracle_lib, t):
    codes = np.arange(256, dtype=np.uint8)
    v = oracle.widen(codes, t)
    for wide in (F32, F16, BF16):
        w = oracle.convert(codes, t, wide)
        back = oracle.convert(w, wide, t)
        fin = np.isfinite(v)
        assert np.array_equal(back[fin], codes[fin]), wide
        assert np.array_equal(oracle.widen(w, wide)[fin], v[fin])


@pytest.mark.parametrize("t", [E4M3, E5M2])
def test_scale_exponent_rule(oracle_lib, t):
    fmax = oracle.FP8_MAX[t]
    assert oracle.fp8_scale_exp(0.0, t) == 0
    assert oracle.fp8_scale_exp(fmax, t) == 0
    assert oracle.fp8_scale_exp(np.nextafter(fmax, np.inf), t) == 1
    assert oracle.fp8_scale_exp(fmax / 2, t) == -1
    assert oracle.fp8_scale_exp(1e300, t) == 126
    assert oracle.fp8_scale_exp(1e-300, t) == -126
    rng = np.random.default_rng(7)
    for a in np.exp2(rng.uniform(-100, 100, 2000)):
        k = oracle.fp8_scale_exp(a, t)
        assert a <= np.ldexp(fmax, k)
        assert a > np.ldexp(fmax, k - 1)


@pytest.mark.parametrize("t", [E4M3, E5M2])
def test_convert_scaled(oracle_lib, t):
    rng = np.random.default_rng(11)
    x = (rng.standard_normal(1 << 16) * 37.5).astype(np.float32)
    x[:5] = [np.inf, -np.inf, np.nan, 0.0, -0.0]
    q, k = oracle.convert_scaled(x, F32, t)
    fin = np.isfinite(x)
    amax = np.abs(x[fin]).max()
    assert k == oracle.fp8_scale_exp(amax, t)
    # codes = the unscaled conversion of x * 2^-k (exact power-of-two scaling)
    want = oracle.convert(np.ldexp(x.astype(np.float64), -k), F64, t)
    assert np.array_equal(q, want)
    # decoding: RNE_f32(code * 2^k) equals the exact value here (no f32 overflow)
    d, k2 = oracle.convert_scaled(q, t, F32, k)
    assert k2 == k
    ex = np.ldexp(oracle.widen(q, t), k)
    dn = np.isnan(ex)
    assert np.array_equal(np.isnan(d), dn)
    assert np.array_equal(d[~dn].astype(np.float64), ex[~dn])
    # the largest finite magnitude uses the top binade: |x| <= FMAX * 2^k
    assert np.abs(ex[np.isfinite(ex)]).max() <= np.ldexp(oracle.FP8_MAX[t], k)
    # relative error of every normal-range element is within half an ulp of the format
    mb = FMT[t][1]
    big = fin & (np.abs(x) >= np.ldexp(2.0 ** (1 - FMT[t][2]), k))
    rel = np.abs(ex[big] - x[big]) / np.abs(x[big])
    assert rel.max() <= 2.0 ** -(mb + 1)


def test_codec_radix6(oracle_lib):
    for m in range(1, 5):
        seen = set()
        for cid in range(6 ** m):
            p = oracle.config_decode(m, cid, radix=6)
            assert oracle.config_encode(p, radix=6) == cid
            seen.add(tuple(p))
        assert len(seen) == 6 ** m
    assert oracle.config_decode(3, 4 + 5 * 6 + 0 * 36, radix=6) == [E4M3, E5M2, F64]


def _small_ints(shape, rng, hi=16):
    return rng.integers(0, hi, size=shape).astype(np.float32)


@pytest.mark.parametrize("ta,tb", [(E4M3, E4M3), (E5M2, E4M3), (E4M3, F16)])
def test_gemm_fp8_exact_integers(oracle_lib, ta, tb):
    """Integers 0..15 (<= 4 significant bits) scale exactly into E4M3, and 0..7 into
    E5M2; with alpha=1, beta=0 and C in f32 the sums are exact: C == A @ B."""
    rng = np.random.default_rng(3)
    NI, NJ, NK = 37, 45, 70
    hi = 8 if E5M2 in (ta, tb) else 16
    A, B = _small_ints((NI, NK), rng, hi), _small_ints((NK, NJ), rng, hi)
    C = np.zeros((NI, NJ), np.float32)
    fin, ks = oracle.run_config("gemm", [NI, NJ, NK], [ta, tb, F32], [A, B, C],
                                scalars=[1.0, 0.0], with_scales=True)
    want = A.astype(np.int64) @ B.astype(np.int64)
    assert np.array_equal(fin[2].astype(np.int64), want)
    for m, t in enumerate([ta, tb]):
        assert np.array_equal(oracle.values(fin[m], t, ks[m]), [A, B][m])


def test_gemm_fp8_output_requantised(oracle_lib):
    """C in E4M3: the exact integer product A @ B re-quantised with the scale of its
    amax, rounded by the brute-force nearest search (independent of oracle.c)."""
    rng = np.random.default_rng(5)
    NI, NJ, NK = 33, 29, 50
    A, B = _small_ints((NI, NK), rng), _small_ints((NK, NJ), rng)
    C = np.zeros((NI, NJ), np.float32)
    fin, ks = oracle.run_config("gemm", [NI, NJ, NK], [F32, F32, E4M3], [A, B, C],
                                scalars=[1.0, 0.0], with_scales=True)
    exact = (A.astype(np.int64) @ B.astype(np.int64)).astype(np.float64)
    amax = exact.max()
    k = int(np.ceil(np.log2(amax / 448.0)))
    assert amax <= 448.0 * 2.0 ** k and amax > 448.0 * 2.0 ** (k - 1)
    assert ks[2] == k
    want = _nearest_fp8(np.ldexp(exact, -k).reshape(-1), E4M3).reshape(NI, NJ)
    assert np.array_equal(fin[2], want)


@pytest.mark.parametrize("kind,dims,prec", [
    ("atax", [300, 260], [E4M3, F32, F32, F32]),
    ("bicg", [270, 300], [E5M2, F32, F32, E4M3, F32]),
    ("mvt", [280], [E4M3, F32, F32, F32, F32]),
])
def test_matvec_fp8_exact_integers(oracle_lib, kind, dims, prec):
    """fp8 matrices holding small integers: every row-dot / column-sum is exact in
    f32, so the result equals exact integer arithmetic (catches dropped or
    duplicated terms and wrong indices in the fp8 decode path)."""
    rng = np.random.default_rng(17)
    objs = oracle.app_objects(kind, dims)
    ins = []
    for o in objs:
        shape = (o["rows"], o["cols"])
        ins.append(_small_ints(shape, rng, 8) if o["role"] in (0, 2) else None)
    fin = oracle.run_config(kind, dims, prec, ins)
    A = ins[0].astype(np.int64)
    if kind == "atax":
        tmp = A @ ins[1].reshape(-1).astype(np.int64)
        want = A.T @ tmp
        assert np.array_equal(fin[2].reshape(-1).astype(np.int64), want)
    elif kind == "bicg":
        s = A.T @ ins[1].reshape(-1).astype(np.int64)
        assert np.array_equal(fin[2].reshape(-1).astype(np.int64), s)
        q = A @ ins[3].reshape(-1).astype(np.int64)      # p (0..7) is exact in E4M3
        assert np.array_equal(fin[4].reshape(-1).astype(np.int64), q)
    else:
        x1 = ins[1].reshape(-1).astype(np.int64) + A @ ins[3].reshape(-1).astype(np.int64)
        x2 = ins[2].reshape(-1).astype(np.int64) + A.T @ ins[4].reshape(-1).astype(np.int64)
        assert np.array_equal(fin[1].reshape(-1).astype(np.int64), x1)
        assert np.array_equal(fin[2].reshape(-1).astype(np.int64), x2)


def test_statement_requantises_whole_object(oracle_lib):
    """FDTD-2D with ey in E5M2: after every ey statement the whole object carries
    one scale, so every stored value is a code * 2^k with |code value| <= 57344."""
    rng = np.random.default_rng(23)
    TM, NX, NY = 3, 20, 24
    ins = [rng.random(TM).astype(np.float32)] + [rng.random((NX, NY)).astype(np.float32)] * 3
    fin, ks = oracle.run_config("fdtd2d", [TM, NX, NY], [F32, F32, E5M2, F32], ins, with_scales=True)
    v = oracle.values(fin[2], E5M2, ks[2])
    assert np.isfinite(v).all()
    amax = np.abs(v).max()
    assert amax <= np.ldexp(57344.0, ks[2])
    # and the run is reproducible against the all-fp64 run within the E5M2 precision
    ref = oracle.reference("fdtd2d", [TM, NX, NY], ins)
    err = np.abs(v - ref[2]) / np.ldexp(1.0, ks[2])
    assert err.max() <= 57344.0 * 2.0 ** -2


def test_quality_fp8_configs_gemm64(oracle_lib):
    """GEMM-64 Random inputs (alpha 1.5, beta 1.2): fp8 inputs lose ~2^-4 per element,
    the contraction averages it out: E4M3 A,B pass TOQ 0.9 and an E5M2-everything
    configuration is worse than E4M3-everything (fewer fraction bits)."""
    from paper_conf_cgo_kangcp20_b200 import inputs as gen
    ins = gen.make_inputs("gemm", oracle.app_objects("gemm", [64]), "random")
    sc = [1.5, 1.2]
    ref = oracle.reference("gemm", [64], ins, sc)
    r43, _ = oracle.evaluate("gemm", [64], [E4M3, E4M3, F32], ins, ref, sc)
    r44, _ = oracle.evaluate("gemm", [64], [E4M3, E4M3, E4M3], ins, ref, sc)
    r55, _ = oracle.evaluate("gemm", [64], [E5M2, E5M2, E5M2], ins, ref, sc)
    assert r43["pass"] and r43["quality"] > 0.97
    assert r55["quality"] < r44["quality"] < r43["quality"]
    assert r44["nonfinite"] == 0 and r55["nonfinite"] == 0
