"""GPU parity of the bf16 object type (reading #28) against
the oracle: conversions bit-exact (every f32 pattern, targeted f64 sets, every
bf16 pattern widened), every radix-4 configuration of the SIMT apps bit-exact,
and the bf16 x bf16 tcgen05 contractions within the R6 bound."""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen
from test_gpu_apps import check_config
from test_gpu_convert import _f64_targets

pytestmark = pytest.mark.gpu
BF = B.BF16


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def _oracle_bf16_mt(x, st):
    import concurrent.futures as cf
    out = np.empty(x.size, dtype=np.uint16)
    b = np.linspace(0, x.size, 9).astype(np.int64)

    def run(i):
        out[b[i]:b[i + 1]] = oracle.convert(x[b[i]:b[i + 1]], st, BF)
    with cf.ThreadPoolExecutor(8) as ex:
        list(ex.map(run, range(8)))
    return out


def test_f32_to_bf16_all_2pow32(torch):
    chunk = 1 << 28
    dst = torch.empty(chunk, dtype=torch.int16, device="cuda")
    for c in range(1 << 4):
        base = c * chunk
        bits = torch.arange(base, base + chunk, dtype=torch.int64, device="cuda")
        bits = (bits - (bits >= 2**31).to(torch.int64) * 2**32).to(torch.int32)
        B.ps_convert(bits.view(torch.float32), B.F32, dst, BF)
        got = dst.cpu().numpy().view(np.uint16)
        x = np.arange(base, base + chunk, dtype=np.uint64).astype(np.uint32).view(np.float32)
        want = _oracle_bf16_mt(x, B.F32)
        bad = np.flatnonzero(got != want)
        assert bad.size == 0, "chunk %d: %d mismatches, first %#x -> %#x want %#x" % (
            c, bad.size, x.view(np.uint32)[bad[0]], got[bad[0]], want[bad[0]])


def test_bf16_widen_and_narrow_all(torch):
    """Every bf16 pattern -> f32 / f64 / f16, and every f16 pattern -> bf16."""
    h = np.arange(1 << 16, dtype=np.uint16)
    src = torch.from_numpy(h.view(np.int16).copy()).cuda()
    for dt, raw in ((B.F32, np.uint32), (B.F64, np.uint64), (B.F16, np.uint16)):
        nbytes = {B.F32: 4, B.F64: 8, B.F16: 2}[dt]
        dst = torch.empty(h.size * nbytes, dtype=torch.uint8, device="cuda")
        B.ps_convert(src.data_ptr(), BF, dst.data_ptr(), dt, h.size)
        torch.cuda.synchronize()
        got = dst.cpu().numpy().view(raw)
        want = oracle.convert(h, BF, dt).view(raw)
        assert np.array_equal(got, want), dt
    hh = torch.from_numpy(h.view(np.int16).copy()).cuda()
    out = torch.empty(h.size, dtype=torch.int16, device="cuda")
    B.ps_convert(hh.data_ptr(), B.F16, out.data_ptr(), BF, h.size)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().view(np.uint16), oracle.convert(h.view(np.float16), B.F16, BF))


def test_f64_to_bf16_single_rounding(torch):
    """Targeted f64 sets + random patterns + the bf16 double-rounding witness."""
    x = np.concatenate([_f64_targets(), np.array([1.0 + 2.0 ** -8 + 2.0 ** -40, -(1.0 + 2.0 ** -8 + 2.0 ** -40),
                                                  2.0 ** 128 - 2.0 ** 119, 2.0 ** -134 * 1.5])])
    src = torch.from_numpy(x.copy()).cuda()
    dst = torch.empty(x.size, dtype=torch.int16, device="cuda")
    B.ps_convert(src, B.F64, dst, BF)
    got = dst.cpu().numpy().view(np.uint16)
    want = _oracle_bf16_mt(x, B.F64)
    bad = np.flatnonzero(got != want)
    assert bad.size == 0, "%d mismatches; first %r -> %#x want %#x" % (bad.size, x[bad[0]], got[bad[0]], want[bad[0]])
    assert got[-4] == 0x3F81


def _setup(torch, kind, dims, iset, sc=None, flags=B.FLAG_BF16 | B.FLAG_NO_TENSOR_CORES):
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
        ("2mm", [40, 50, 30, 20], "random", None)]


@pytest.mark.parametrize("kind,dims,iset,sc", SIMT, ids=[c[0] for c in SIMT])
def test_radix4_configs_bit_exact_simt(torch, kind, dims, iset, sc):
    """Every configuration containing bf16 (sampled to 200), bit-exact delivered
    outputs, max error and non-finite count; quality within 1e-12 (its fp64
    summation order differs)."""
    app, ins, oref = _setup(torch, kind, dims, iset, sc)
    m = app.num_objects
    assert app.space == 4 ** m
    ids = [c for c in range(app.space) if BF in app.decode(c)]
    if len(ids) > 200:
        ids = sorted(np.random.default_rng(1).choice(ids, 200, replace=False).tolist())
    for cid in ids:
        prec = app.decode(cid)
        assert prec == oracle.config_decode(m, cid, 4)
        check_config(torch, app, kind, dims, ins, oref, prec, sc)   # bit-exact outputs


def test_radix4_sweep_and_best(torch):
    """ps_sweep over all 4^3 GEMM configurations == one run each; best = fastest passing."""
    app, ins, oref = _setup(torch, "gemm", [64], "random", (1.5, 1.2))
    ids = list(range(app.space))
    arr, best = app.sweep_raw(ids, 0.9)
    assert list(arr["config_id"]) == ids and best >= 0
    for cid in (0, 21, 42, 63):
        r = app.run_config(app.decode(cid))
        assert r["quality"] == arr["quality"][cid]
    with pytest.raises(B.PsError):
        app.decode(64)
    app.set_flags(B.FLAG_NO_TENSOR_CORES)        # back to the paper's 3^M alphabet
    assert app.space == 27
    with pytest.raises(B.PsError):
        app.run_config([BF, 1, 1])


def gamma(k):
    u = 2.0 ** -24
    return k * u / (1 - k * u)


@pytest.mark.parametrize("dims", [[264, 136, 520], [300, 200, 129]])
def test_gemm_bf16_tensor_core_bound(torch, dims):
    """bf16 x bf16 on tcgen05 (kind::f16, bf16 operand format), C in f32 / bf16."""
    sc = (1.5, 1.2)
    app, ins, oref = _setup(torch, "gemm", dims, "random", sc, flags=B.FLAG_BF16)
    for cprec in (B.F32, BF):
        prec = [BF, BF, cprec]
        r = app.run_config(prec)
        ro, delivered = oracle.evaluate("gemm", dims, prec, ins, oref, sc)
        got = app.outputs[2].cpu().numpy().astype(np.float64).reshape(dims[0], dims[1])
        want = delivered[2].astype(np.float64).reshape(dims[0], dims[1])
        st = oracle.run_config("gemm", dims, prec, ins, sc)
        a = np.abs(oracle.widen(st[0], BF).reshape(dims[0], dims[2]))
        b = np.abs(oracle.widen(st[1], BF).reshape(dims[2], dims[1]))
        ulp_c = 2.0 ** -7 if cprec == BF else 2.0 ** -23
        bound = sc[0] * 2 * gamma(dims[2]) * (a @ b) + 2 * ulp_c * np.abs(want) + 1e-30
        assert np.all(np.abs(got - want) <= bound), cprec
        assert abs(r["quality"] - ro["quality"]) <= 1e-3
