"""GPU parity of the tcgen05 tensor-core contraction path (reading R6).

Statements with two fp16 multiplicands and compute type f32 run on tcgen05
(UTCHMMA); the accumulation order inside the tensor core is unspecified, so the
delivered outputs are compared with the oracle within the error bound
    |gpu - oracle| <= s * 2 gamma_K(2^-24) * sum_k |a_k b_k| + 2 ulp(out)
(s = |alpha| or 1/(n-1) of the epilogue), computed from the fp16 operands the
oracle actually stores.  Chained statements (2MM/3MM) use the north-star bound:
<= 2^-10 relative per element for fp16 objects on positive inputs.
"""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

pytestmark = pytest.mark.gpu
U = 2.0 ** -24


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def gamma(k):
    return k * U / (1 - k * U)


def setup(torch, kind, dims, iset, scalars=None):
    app = B.App(kind, dims, scalars)
    app.set_flags(0)                           # tensor cores enabled
    ins = gen.make_inputs(kind, app.objects, iset)
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    oref = oracle.reference(kind, dims, ins, scalars)
    return app, ins, oref


def ulp(x, dtype):
    return np.spacing(np.abs(x).astype(dtype)).astype(np.float64)


@pytest.mark.parametrize("dims,iset,sc", [([200, 264, 136], "random", (1.5, 1.2)),
                                          ([128, 256, 64], "random", (1.5, 1.2)),
                                          ([520, 776, 1048], "image", (0.5, -0.25)),
                                          ([64, 64, 64], "default", None)])
@pytest.mark.parametrize("c_prec", [B.F32, B.F16])
def test_gemm_tc_bound(torch, dims, iset, sc, c_prec):
    app, ins, oref = setup(torch, "gemm", dims, iset, sc)
    prec = [B.F16, B.F16, c_prec]
    r = app.run_config(prec)
    ro, delivered = oracle.evaluate("gemm", dims, prec, ins, oref, sc)
    got = app.outputs[2].cpu().numpy().astype(np.float64)
    want = delivered[2].reshape(-1).astype(np.float64)
    fin = oracle.run_config("gemm", dims, prec, ins, sc)
    a16, b16 = fin[0].astype(np.float64), fin[1].astype(np.float64)
    al = (sc or (32412.0, 2123.0))[0]
    bound = abs(al) * 2 * gamma(dims[2]) * (np.abs(a16) @ np.abs(b16)).reshape(-1)
    bound += 2 * ulp(want, np.float16 if c_prec == B.F16 else np.float32)
    finite = np.isfinite(want)
    assert np.array_equal(np.isfinite(got), finite)
    err = np.abs(got[finite] - want[finite])
    assert np.all(err <= bound[finite]), (err.max(), (err / bound[finite]).max())
    assert r["nonfinite"] == ro["nonfinite"]
    assert abs(r["quality"] - ro["quality"]) <= 1e-3


@pytest.mark.parametrize("kind,dims,prec", [
    ("covar", [264, 136], [B.F16, B.F32, B.F32]),
    ("covar", [512, 520], [B.F16, B.F16, B.F16]),
    ("corr", [300, 136], [B.F16, B.F32, B.F32, B.F32]),
    ("corr", [257, 264], [B.F16, B.F16, B.F16, B.F16]),
])
def test_syrk_tc_bound(torch, kind, dims, prec):
    """SYRK on tcgen05 with the M-major A operand (data^T), upper tiles + mirror."""
    app, ins, oref = setup(torch, kind, dims, "random")
    r = app.run_config(prec)
    ro, delivered = oracle.evaluate(kind, dims, prec, ins, oref)
    so = 3 if kind == "corr" else 2
    got = app.outputs[so].cpu().numpy().astype(np.float64).reshape(dims[1], dims[1])
    want = delivered[so].astype(np.float64).reshape(dims[1], dims[1])
    fin = oracle.run_config(kind, dims, prec, ins)
    d = np.abs(fin[0].astype(np.float64))          # the fp16 operand after the earlier statements
    scale = 1.0 if kind == "corr" else 1.0 / (dims[0] - 1)
    bound = scale * 2 * gamma(dims[0]) * (d.T @ d) + 2 * ulp(want, np.float16 if prec[-1] == B.F16 else np.float32)
    assert np.array_equal(got, got.T)
    err = np.abs(got - want)
    assert np.all(err <= bound), ((err - bound).max(), np.unravel_index(np.argmax(err - bound), err.shape))
    assert abs(r["quality"] - ro["quality"]) <= 1e-3


@pytest.mark.parametrize("dims,c_prec", [([264, 136], B.F32), ([520, 264], B.F16)])
def test_syrk_app_tc_bound(torch, dims, c_prec):
    """SYRK app: C <- alpha A^T A + beta C on tcgen05 (A fp16, M-major operand)."""
    sc = (1.5, 1.2)
    app, ins, oref = setup(torch, "syrk", dims, "random", sc)
    prec = [B.F16, c_prec]
    r = app.run_config(prec)
    ro, delivered = oracle.evaluate("syrk", dims, prec, ins, oref, sc)
    M = dims[1]
    got = app.outputs[1].cpu().numpy().astype(np.float64).reshape(M, M)
    want = delivered[1].astype(np.float64).reshape(M, M)
    a16 = np.abs(oracle.run_config("syrk", dims, prec, ins, sc)[0].astype(np.float64))
    bound = sc[0] * 2 * gamma(dims[0]) * (a16.T @ a16) + 2 * ulp(want, np.float16 if c_prec == B.F16 else np.float32)
    assert np.array_equal(got, got.T)
    assert np.all(np.abs(got - want) <= bound)
    assert abs(r["quality"] - ro["quality"]) <= 1e-3


@pytest.mark.parametrize("dims,c_prec", [([264, 136], B.F32), ([200, 264], B.F16)])
def test_syr2k_app_tc_bound(torch, dims, c_prec):
    """SYR2K app (reading #25): two tcgen05 statements into the same C.  Each
    statement contributes its gamma_K bound; C is rounded once per statement."""
    sc = (1.5, 1.2)
    app, ins, oref = setup(torch, "syr2k", dims, "random", sc)
    prec = [B.F16, B.F16, c_prec]
    r = app.run_config(prec)
    ro, delivered = oracle.evaluate("syr2k", dims, prec, ins, oref, sc)
    M = dims[1]
    got = app.outputs[2].cpu().numpy().astype(np.float64).reshape(M, M)
    want = delivered[2].astype(np.float64).reshape(M, M)
    st = oracle.run_config("syr2k", dims, prec, ins, sc)
    a16 = np.abs(st[0].astype(np.float64).reshape(dims[0], M))
    b16 = np.abs(st[1].astype(np.float64).reshape(dims[0], M))
    u = ulp(want, np.float16 if c_prec == B.F16 else np.float32)
    bound = sc[0] * 2 * gamma(dims[0]) * (a16.T @ b16 + b16.T @ a16) * (1 + 2 ** -10) + 4 * u
    assert np.all(np.abs(got - want) <= bound)
    assert abs(r["quality"] - ro["quality"]) <= 1e-3


@pytest.mark.parametrize("kind,dims", [("2mm", [136, 264, 200, 72]), ("3mm", [136, 72, 200, 64, 128])])
def test_chain_tc_relative(torch, kind, dims):
    """Every config of the chain apps with tensor cores enabled: fp16 statements
    within 2^-10 relative per element of the oracle (positive random inputs)."""
    app, ins, oref = setup(torch, kind, dims, "random")
    step = 1 if kind == "2mm" else 7
    for cid in range(0, app.space, step):
        prec = app.decode(cid)
        r = app.run_config(prec)
        ro, delivered = oracle.evaluate(kind, dims, prec, ins, oref)
        out = len(prec) - 1
        got = app.outputs[out].cpu().numpy().astype(np.float64)
        want = delivered[out].reshape(-1).astype(np.float64)
        fin = np.isfinite(want)
        assert np.array_equal(np.isfinite(got), fin)
        rel = np.abs(got[fin] - want[fin]) / np.maximum(np.abs(want[fin]), 1e-300)
        assert np.all(rel <= 2.0 ** -10), (prec, rel.max())
        assert abs(r["quality"] - ro["quality"]) <= 2.0 ** -10


def test_tc_and_simt_agree_on_pass_set(torch):
    """GEMM-64 (config 1): the TOQ pass set is the same with and without tensor cores."""
    app, ins, oref = setup(torch, "gemm", [64], "default")
    res_tc, _ = app.sweep(range(27))
    app.set_flags(B.FLAG_NO_TENSOR_CORES)
    res_simt, _ = app.sweep(range(27))
    assert [r["pass"] for r in res_tc] == [r["pass"] for r in res_simt]
