"""GPU parity of the fp8 object types (reading #29)
against the oracle: unscaled conversions bit-exact over every f32 pattern and
targeted f64 sets, every code decoded at several scales, scaled conversions
(amax -> k -> codes) bit-exact, every radix-6 configuration of the SIMT apps
(sampled) bit-exact, and the fp8 x fp8 tcgen05 (kind::f8f6f4) contractions
within the R6 bound."""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen
from test_gpu_apps import check_config

pytestmark = pytest.mark.gpu
E4, E5 = B.E4M3, B.E5M2
RAW = {B.F64: np.uint64, B.F32: np.uint32, B.F16: np.uint16, B.BF16: np.uint16}
SIZE = {B.F64: 8, B.F32: 4, B.F16: 2, B.BF16: 2, E4: 1, E5: 1}


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def _oracle_mt(x, st, dt):
    import concurrent.futures as cf
    out = np.empty(x.size, dtype=oracle.NP_DTYPE[dt])
    b = np.linspace(0, x.size, 17).astype(np.int64)

    def run(i):
        out[b[i]:b[i + 1]] = oracle.convert(x[b[i]:b[i + 1]], st, dt)
    with cf.ThreadPoolExecutor(16) as ex:
        list(ex.map(run, range(16)))
    return out


@pytest.mark.parametrize("t", [E4, E5])
def test_f32_to_fp8_all_2pow32_unscaled(torch, t):
    chunk = 1 << 28
    dst = torch.empty(chunk, dtype=torch.uint8, device="cuda")
    for c in range(1 << 4):
        base = c * chunk
        bits = torch.arange(base, base + chunk, dtype=torch.int64, device="cuda")
        bits = (bits - (bits >= 2**31).to(torch.int64) * 2**32).to(torch.int32)
        B.ps_convert(bits.view(torch.float32), B.F32, dst, t)
        got = dst.cpu().numpy()
        x = np.arange(base, base + chunk, dtype=np.uint64).astype(np.uint32).view(np.float32)
        want = _oracle_mt(x, B.F32, t)
        bad = np.flatnonzero(got != want)
        assert bad.size == 0, "chunk %d: %d mismatches, first %#x -> %#x want %#x" % (
            c, bad.size, x.view(np.uint32)[bad[0]], got[bad[0]], want[bad[0]])


def _f64_fp8_targets(t):
    vals = np.unique(np.abs(oracle.widen(np.arange(128, dtype=np.uint8), t)))
    vals = vals[np.isfinite(vals)]
    mids = np.concatenate([(vals[:-1] + vals[1:]) / 2, [vals[-1] + (vals[-1] - vals[-2]) / 2]])
    cand = [mids, vals]
    up, dn = mids.copy(), mids.copy()
    for _ in range(4):
        up, dn = np.nextafter(up, np.inf), np.nextafter(dn, -np.inf)
        cand += [up, dn]
    rng = np.random.default_rng(5)
    cand += [rng.uniform(0, 1.3 * vals[-1], 1 << 20), np.exp2(rng.uniform(-30, 20, 1 << 20)),
             rng.integers(0, 2**64, 1 << 20, dtype=np.uint64).view(np.float64),
             np.array([np.inf, -np.inf, np.nan, 0.0, -0.0, 1e300, -1e-300])]
    x = np.concatenate(cand)
    return np.concatenate([x, -x])


@pytest.mark.parametrize("t", [E4, E5])
def test_f64_to_fp8_single_rounding_unscaled(torch, t):
    x = _f64_fp8_targets(t)
    src = torch.from_numpy(x.copy()).cuda()
    dst = torch.empty(x.size, dtype=torch.uint8, device="cuda")
    B.ps_convert(src, B.F64, dst, t)
    got = dst.cpu().numpy()
    want = oracle.convert(x, B.F64, t)
    bad = np.flatnonzero(got != want)
    assert bad.size == 0, "%d mismatches; first %r -> %#x want %#x" % (bad.size, x[bad[0]], got[bad[0]], want[bad[0]])


@pytest.mark.parametrize("t", [E4, E5])
def test_fp8_decode_all_codes_scaled(torch, t):
    codes = np.tile(np.arange(256, dtype=np.uint8), 3)    # vector body + ragged tail
    src = torch.from_numpy(codes).cuda()
    scale = torch.zeros(16, dtype=torch.uint8, device="cuda")
    for k in (-126, -40, -7, 0, 5, 60, 126):
        scale.view(torch.int32)[2] = k
        for dt in (B.F64, B.F32, B.F16, B.BF16):
            dst = torch.empty(codes.size * SIZE[dt], dtype=torch.uint8, device="cuda")
            B.ps_convert_scaled(src, t, dst, dt, scale, n=codes.size)
            torch.cuda.synchronize()
            got = dst.cpu().numpy().view(RAW[dt])
            want, _ = oracle.convert_scaled(codes, t, dt, k)
            assert np.array_equal(got, want.view(RAW[dt])), (k, dt)


@pytest.mark.parametrize("t", [E4, E5])
@pytest.mark.parametrize("st", [B.F32, B.F64, B.F16, B.BF16])
def test_fp8_encode_scaled(torch, t, st):
    """amax over the finite values -> k -> RNE_fp8(x * 2^-k), bit-exact with the oracle,
    for several magnitude ranges (k from -126 to 126), NaN/inf and ragged n."""
    rng = np.random.default_rng(st * 10 + t)
    for mag in (1e-30, 3e-3, 1.0, 448.0, 7e4, 1e30):
        n = 100003
        x = rng.standard_normal(n) * mag
        x[:6] = [np.inf, -np.inf, np.nan, 0.0, -0.0, mag * 1e-6]
        if st == B.F16:
            x = np.clip(x, -65504, 65504)
            xs = x.astype(np.float16)
        elif st == B.BF16:
            xs = oracle.convert(x.astype(np.float32), B.F32, B.BF16)
        elif st == B.F32:
            xs = x.astype(np.float32)
        else:
            xs = x
        src = torch.from_numpy(xs.view(RAW[st]).view(np.int64 if st == B.F64 else
                                                      (np.int32 if st == B.F32 else np.int16)).copy()).cuda()
        dst = torch.empty(n, dtype=torch.uint8, device="cuda")
        scale = torch.zeros(16, dtype=torch.uint8, device="cuda")
        B.ps_convert_scaled(src, st, dst, t, scale, n=n)
        torch.cuda.synchronize()
        want, kw = oracle.convert_scaled(xs, st, t)
        k = int(scale.cpu().numpy().view(np.int32)[2])
        assert k == kw, (mag, k, kw)
        got = dst.cpu().numpy()
        bad = np.flatnonzero(got != want)
        assert bad.size == 0, (mag, bad.size, got[bad[0]], want[bad[0]])


def _setup(torch, kind, dims, iset, sc=None, flags=B.FLAG_FP8 | B.FLAG_NO_TENSOR_CORES):
    app = B.App(kind, dims, sc)
    app.set_flags(flags)
    ins = gen.make_inputs(kind, app.objects, iset)
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    oref = oracle.reference(kind, dims, ins, sc)
    return app, ins, oref


SIMT = [("gemm", [70, 66, 33], "random", (1.5, 1.2)), ("atax", [517, 333], "random", None),
        ("bicg", [301, 257], "random", None), ("gesummv", [301], "random", None),
        ("corr", [130, 70], "random", None), ("covar", [130, 45], "random", None),
        ("mvt", [600], "random", None), ("syrk", [129, 70], "random", (1.5, 1.2)),
        ("conv2d", [70, 130], "image", None), ("syr2k", [66, 40], "random", (1.5, 1.2)),
        ("conv3d", [12, 20, 70], "random", None), ("fdtd2d", [3, 40, 70], "random", None),
        ("2mm", [40, 50, 30, 20], "random", None), ("3mm", [20, 24, 28, 32, 36], "random", None),
        ("atax", [300, 200], "default", None), ("gemm", [64], "default", None)]


@pytest.mark.parametrize("kind,dims,iset,sc", SIMT, ids=["%s-%s" % (c[0], c[2]) for c in SIMT])
def test_radix6_configs_bit_exact_simt(torch, kind, dims, iset, sc):
    """Configurations containing fp8 objects (sampled to 80 per app, always including
    the uniform E4M3 / E5M2 ones), SIMT path: delivered outputs, max error and
    non-finite count bit-exact; quality within 1e-12."""
    app, ins, oref = _setup(torch, kind, dims, iset, sc)
    m = app.num_objects
    assert app.space == 6 ** m
    ids = [c for c in range(app.space) if any(p >= E4 for p in app.decode(c))]
    uni = [app.encode([E4] * m), app.encode([E5] * m)]
    rng = np.random.default_rng(2)
    if len(ids) > 80:
        ids = sorted(set(rng.choice(ids, 78, replace=False).tolist()) | set(uni))
    for cid in ids:
        prec = app.decode(cid)
        assert prec == oracle.config_decode(m, cid, 6)
        check_config(torch, app, kind, dims, ins, oref, prec, sc)


def gamma(k, u=2.0 ** -24):
    return k * u / (1 - k * u)


def _fp8_vals(st, t, k):
    return np.ldexp(oracle.widen(st, t), k)


@pytest.mark.parametrize("dims,ta,tb", [([264, 136, 520], E4, E4), ([300, 200, 129], E5, E4),
                                        ([520, 600, 1000], E4, E5), ([64, 64, 64], E5, E5)])
def test_gemm_fp8_tensor_core_bound(torch, dims, ta, tb):
    """fp8 x fp8 on tcgen05 (kind::f8f6f4): C in f32 within the R6 bound of the
    oracle's f32 chain; C in E4M3 within one E4M3 quantum of it."""
    sc = (1.5, 1.2)
    app, ins, oref = _setup(torch, "gemm", dims, "random", sc, flags=B.FLAG_FP8)
    for cprec in (B.F32, E4):
        prec = [ta, tb, cprec]
        r = app.run_config(prec)
        ro, delivered = oracle.evaluate("gemm", dims, prec, ins, oref, sc)
        got = app.outputs[2].cpu().numpy().astype(np.float64).reshape(dims[0], dims[1])
        want = delivered[2].astype(np.float64).reshape(dims[0], dims[1])
        st, ks = oracle.run_config("gemm", dims, prec, ins, sc, with_scales=True)
        a = np.abs(_fp8_vals(st[0], ta, ks[0]).reshape(dims[0], dims[2]))
        b = np.abs(_fp8_vals(st[1], tb, ks[1]).reshape(dims[2], dims[1]))
        bound = sc[0] * 2 * gamma(dims[2]) * (a @ b) + 2 * 2.0 ** -23 * np.abs(want) + 1e-30
        if cprec == E4:    # a re-quantised output: one quantum of the output's scale
            bound = bound + np.ldexp(2.0 ** -3, int(np.floor(np.log2(np.abs(want).max())))) + 1e-30
        err = np.abs(got - want)
        assert np.all(err <= bound), (cprec, float((err / np.maximum(bound, 1e-300)).max()))
        assert abs(r["quality"] - ro["quality"]) <= 2e-3


@pytest.mark.parametrize("kind,dims", [("syrk", [520, 300]), ("covar", [600, 264]), ("syr2k", [260, 136]),
                                       ("2mm", [300, 260, 200, 136])])
def test_fp8_tensor_core_apps(torch, kind, dims):
    """M-major fp8 A (SYRK/COVAR data^T, SYR2K), chained 2MM: quality of the fp8
    tensor-core configurations within 2e-3 of the oracle's (R6)."""
    sc = (1.5, 1.2) if kind in ("syrk", "syr2k") else None
    app, ins, oref = _setup(torch, kind, dims, "random", sc, flags=B.FLAG_FP8)
    m = app.num_objects
    for prec in ([E4] * m, [E5] * m, [E4 if i < m - 1 else B.F32 for i in range(m)]):
        r = app.run_config(prec)
        ro, _ = oracle.evaluate(kind, dims, prec, ins, oref, sc)
        assert r["nonfinite"] == ro["nonfinite"]
        assert abs(r["quality"] - ro["quality"]) <= 2e-3, (prec, r["quality"], ro["quality"])


def test_radix6_sweep_search(torch):
    """ps_sweep over all 6^3 GEMM-64 configurations == one run each; ps_search with
    the fp8 alphabet ends on a passing configuration at least as fast as PFP's."""
    app, ins, oref = _setup(torch, "gemm", [64], "random", (1.5, 1.2), flags=B.FLAG_FP8)
    ids = list(range(app.space))
    arr, best = app.sweep_raw(ids, 0.9)
    assert list(arr["config_id"]) == ids and best >= 0
    for cid in (0, 4 + 4 * 6 + 1 * 36, 215):
        r = app.run_config(app.decode(cid))
        assert abs(r["quality"] - arr["quality"][cid]) <= 1e-12
    s = app.search(0.9)
    assert s["pass"] and s["trials"] >= 6
    with pytest.raises(B.PsError):
        app.decode(216)


def test_fp8_flag_after_bind_rejected(torch):
    app, ins, oref = _setup(torch, "gemm", [32], "random", (1.5, 1.2), flags=B.FLAG_NO_TENSOR_CORES)
    with pytest.raises(B.PsError):
        app.set_flags(B.FLAG_FP8)
    with pytest.raises(B.PsError):
        app.run_config([E4, 1, 1])
