"""GPU parity of the whole configuration evaluation (rows a0-a7) vs the oracle.

Every configuration of every app, at sizes spanning several tiles / chunks with
ragged tails, on both aligned and unaligned row strides.  SIMT paths
(PS_FLAG_NO_TENSOR_CORES, and every config without two fp16 multiplicands) are
BIT-EXACT with the oracle on the delivered outputs and the fp64 reference
(readings R3/R5); max_rel and the non-finite count are exact; Q within 1e-12
(the oracle sums e sequentially, the GPU with a fixed tree, c-5).
"""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def same_bits(a: np.ndarray, b: np.ndarray) -> bool:
    a = np.ascontiguousarray(a).reshape(-1)
    b = np.ascontiguousarray(b).reshape(-1)
    if a.shape != b.shape:
        return False
    raw = {4: np.uint32, 8: np.uint64}[a.dtype.itemsize]
    eq = a.view(raw) == b.view(raw)
    both_nan = np.isnan(a) & np.isnan(b)
    return bool(np.all(eq | both_nan))


def setup_app(torch, kind, dims, iset, scalars=None, flags=B.FLAG_NO_TENSOR_CORES, seed=0):
    app = B.App(kind, dims, scalars)
    app.set_flags(flags)
    ins = gen.make_inputs(kind, app.objects, iset, seed)
    dins = [torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins]
    app.bind(dins)
    refs = app.reference()
    oref = oracle.reference(kind, dims, ins, scalars)
    for m, o in enumerate(app.objects):
        if o["is_output"]:
            assert same_bits(refs[m].cpu().numpy(), oref[m]), "fp64 reference differs (obj %d)" % m
    return app, ins, oref


def check_config(torch, app, kind, dims, ins, oref, prec, scalars=None, toq=0.9, exact=True,
                 rtol=None):
    r = app.run_config(prec, toq)
    ro, delivered = oracle.evaluate(kind, dims, prec, ins, oref, scalars, toq)
    for m, o in enumerate(app.objects):
        if not o["is_output"]:
            continue
        got = app.outputs[m].cpu().numpy()
        want = delivered[m].reshape(-1)
        if exact:
            if not same_bits(got, want):
                bad = np.flatnonzero(~((got.view(np.uint32) == want.view(np.uint32)) |
                                       (np.isnan(got) & np.isnan(want))))
                raise AssertionError("%s prec=%s obj %s: %d/%d elements differ, first at %d: "
                                     "gpu %r oracle %r" % (kind, prec, o["name"], bad.size, got.size,
                                                           bad[0], got[bad[0]], want[bad[0]]))
        else:
            fin = np.isfinite(want)
            assert np.array_equal(np.isfinite(got), fin)
            np.testing.assert_allclose(got[fin], want[fin], rtol=rtol,
                                       atol=rtol * np.abs(want[fin]).max() if fin.any() else 0)
    if exact:
        assert r["nonfinite"] == ro["nonfinite"], (prec, r, ro)
        assert r["max_rel"] == ro["max_rel"] or (np.isnan(r["max_rel"]) and np.isnan(ro["max_rel"]))
        assert abs(r["quality"] - ro["quality"]) <= 1e-12, (prec, r["quality"], ro["quality"])
        if abs(ro["quality"] - toq) > 1e-9:
            assert r["pass"] == ro["pass"]
    assert r["status"] == 0 and r["config_id"] == app.encode(prec)
    assert r["total_ms"] >= 0 and r["kernel_ms"] >= 0
    return r, ro


SIMT_CASES = [
    ("gemm", [200, 150, 70], "default", None),
    ("gemm", [129, 66, 33], "random", (1.5, 1.2)),
    ("2mm", [130, 70, 90, 45], "random", None),
    ("2mm", [70, 40, 33, 65], "default", None),
    ("atax", [600, 336], "default", None),
    ("atax", [517, 333], "random", None),
    ("bicg", [700, 344], "default", None),
    ("bicg", [301, 257], "random", None),
    ("gesummv", [304], "default", None),
    ("gesummv", [301], "random", None),
    ("corr", [300, 70], "random", None),
    ("corr", [257, 33], "image", None),
    ("covar", [260, 90], "random", None),
    ("covar", [511, 37], "default", None),
    ("mvt", [600], "random", None),
    ("mvt", [2051], "default", None),
    ("syrk", [260, 70], "random", (1.5, 1.2)),
    ("syrk", [129, 257], "default", None),
    ("conv2d", [200, 300], "random", None),
    ("conv2d", [37, 65], "image", None),
    ("syr2k", [260, 70], "random", (1.5, 1.2)),
    ("syr2k", [67, 130], "default", None),
    ("conv3d", [20, 30, 70], "random", None),
    ("conv3d", [9, 17, 300], "image", None),
    ("fdtd2d", [5, 130, 70], "random", None),
    ("fdtd2d", [20, 33, 301], "default", None),
]


@pytest.mark.parametrize("kind,dims,iset,sc", SIMT_CASES,
                         ids=["%s-%s-%s" % (c[0], "x".join(map(str, c[1])), c[2]) for c in SIMT_CASES])
def test_every_config_bit_exact_simt(torch, kind, dims, iset, sc):
    app, ins, oref = setup_app(torch, kind, dims, iset, sc)
    for cid in range(app.space):
        check_config(torch, app, kind, dims, ins, oref, app.decode(cid), sc)


def test_3mm_every_config_bit_exact_simt(torch):
    kind, dims = "3mm", [40, 50, 30, 60, 20]
    app, ins, oref = setup_app(torch, kind, dims, "random")
    for cid in range(app.space):
        check_config(torch, app, kind, dims, ins, oref, app.decode(cid))


@pytest.mark.parametrize("kind,dims", [("gemm", [64]), ("atax", [600, 336]), ("corr", [300, 70])])
def test_sweep_equals_individual_runs(torch, kind, dims):
    """Exhaustive enumeration (one ps_run_config per id) == ps_sweep over all ids,
    and == the oracle's sweep on the passing set (north star invariant)."""
    app, ins, oref = setup_app(torch, kind, dims, "random" if kind == "corr" else "default")
    ids = list(range(app.space))
    res, best = app.sweep(ids, 0.9)
    _, ores = oracle.sweep(kind, dims, ids, ins, ref=oref, toq=0.9)
    for cid, r, ro in zip(ids, res, ores):
        single = app.run_config(app.decode(cid), 0.9)
        assert r["config_id"] == cid
        assert r["quality"] == single["quality"] and r["max_rel"] == single["max_rel"]
        assert r["nonfinite"] == ro["nonfinite"] and abs(r["quality"] - ro["quality"]) <= 1e-12
        assert r["pass"] == ro["pass"]
    passing = [i for i, r in enumerate(res) if r["pass"]]
    if passing:
        tmin = min(res[i]["total_ms"] for i in passing)
        assert res[best]["pass"] and res[best]["total_ms"] == tmin
        assert best == min(i for i in passing if res[i]["total_ms"] == tmin)
    else:
        assert best == -1


def test_gemm64_config1_pass_set(torch):
    """BASELINE config 1: GEMM N=64, 27 configs, TOQ 0.9: 18 pass (C in fp16 overflows)."""
    app, ins, oref = setup_app(torch, "gemm", [64], "default", flags=0)
    res, best = app.sweep(range(27), 0.9)
    passing = {r["config_id"] for r in res if r["pass"]}
    assert passing == {c for c in range(27) if app.decode(c)[2] != B.F16}
    assert best >= 0 and res[best]["pass"]


def test_ps_quality_standalone(torch):
    rng = np.random.default_rng(1)
    ref = rng.standard_normal(100003) * 10
    for t, dt in [(0, np.float64), (1, np.float32), (2, np.float16)]:
        out = ref.astype(dt)
        out[17] = np.inf
        g = B.ps_quality(torch.from_numpy(out).cuda(), t, torch.from_numpy(ref).cuda())
        o = oracle.quality(out, t, ref)
        assert g["nonfinite"] == o["nonfinite"] == 1
        assert g["max_rel"] == o["max_rel"]
        assert abs(g["quality"] - o["quality"]) <= 1e-12
        g2 = B.ps_quality(torch.from_numpy(out).cuda(), t, torch.from_numpy(ref).cuda(),
                          metric=B.METRIC_MAX_REL)
        assert g2["quality"] == 0.0


def test_load_host_roundtrip(torch):
    """e2e path: host inputs copied through ps_app_load_host give the same results."""
    kind, dims = "bicg", [301, 257]
    app, ins, oref = setup_app(torch, kind, dims, "random")
    r1 = app.run_config([1, 2, 0, 1, 2])
    for t in app.inputs:
        if t is not None:
            t.zero_()
    host = [torch.from_numpy(a.reshape(-1)).pin_memory() if a is not None else None for a in ins]
    app.load_host(host)
    r2 = app.run_config([1, 2, 0, 1, 2])
    assert r1["quality"] == r2["quality"] and r1["max_rel"] == r2["max_rel"]
