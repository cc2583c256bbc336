"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (ps_app_bind + ps_run_config, same kernels as ps_sweep), on outputs the
oracle computes one by one (oracle.sample).

SIMT / mat-vec statements: bit-exact on the sampled delivered outputs (and on the
fp64 reference).  Tensor-core (fp16 x fp16) statements: 2^-10 relative per
element for positive inputs (north star), reading R6.
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


def f32_bits(x64):
    """RNE to f32 of raw values (the a4 back-conversion), via the oracle converter."""
    return oracle.convert(np.ascontiguousarray(x64, dtype=np.float64), 0, 1).view(np.uint32)


def run(torch, kind, dims, iset, configs, samples, tc_rel=None, flags=0):
    app = B.App(kind, dims)
    app.set_flags(flags)
    ins = gen.make_inputs(kind, app.objects, iset)
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    refs = app.reference()
    m_obj = len(app.objects)
    # the fp64 reference (config 0), bit-exact on the samples
    for k, (rows, cols) in samples.items():
        want = oracle.sample(kind, dims, [0] * m_obj, ins, k, rows, cols)
        got = refs[k].view(app.objects[k]["rows"], app.objects[k]["cols"])[rows, cols].cpu().numpy()
        assert np.array_equal(got.view(np.uint64), want.view(np.uint64)), (kind, "reference", k)
    for prec in configs:
        app.run_config(prec)
        torch.cuda.synchronize()
        for k, (rows, cols) in samples.items():
            o = app.objects[k]
            raw = oracle.sample(kind, dims, prec, ins, k, rows, cols)
            got = app.outputs[k].view(o["rows"], o["cols"])[rows, cols].cpu().numpy()
            exact = tc_rel is None or not tc_rel(prec)
            if exact:
                want = f32_bits(raw)
                ok = (got.view(np.uint32) == want) | (np.isnan(got) & np.isnan(raw))
                assert np.all(ok), (kind, prec, k, np.flatnonzero(~ok)[:5], got[~ok][:3], raw[~ok][:3])
            else:
                fin = np.isfinite(raw)
                assert np.array_equal(np.isfinite(got), fin), (kind, prec, k)
                rel = np.abs(got[fin] - raw[fin]) / np.maximum(np.abs(raw[fin]), 1e-300)
                assert np.all(rel <= 2.0 ** -10), (kind, prec, k, rel.max())


def _vec_samples(n, rng, cnt=256):
    idx = np.sort(rng.choice(n, size=cnt, replace=False))
    return np.zeros(cnt, dtype=np.int64), idx


MV_CONFIGS = {
    4: [[1, 1, 1, 1], [2, 2, 2, 2], [2, 1, 0, 2], [0, 2, 1, 1]],
    5: [[1, 1, 1, 1, 1], [2, 2, 2, 2, 2], [2, 1, 0, 2, 1], [0, 2, 1, 1, 2]],
}


@pytest.mark.parametrize("kind,dims,outs", [("bicg", [16384, 16384], [2, 4]),
                                            ("gesummv", [16384], [3]),
                                            ("atax", [16384, 16384], [2])])
def test_matvec_n16384(torch, kind, dims, outs):
    rng = np.random.default_rng(0)
    n = dims[-1] if kind != "gesummv" else dims[0]
    samples = {k: _vec_samples(n, rng) for k in outs}
    nobj = 4 if kind == "atax" else 5
    cfgs = MV_CONFIGS[nobj] if kind != "atax" else MV_CONFIGS[4][:2]
    run(torch, kind, dims, "default", cfgs, samples)


def _mat_samples(rows, cols, rng, nr=2, nc=8):
    r = np.sort(rng.choice(rows, size=nr, replace=False))
    c = np.sort(rng.choice(cols, size=nc, replace=False))
    rr, cc = np.meshgrid(r, c, indexing="ij")
    return rr.reshape(-1), cc.reshape(-1)


def _tc_chain(prec):
    # a statement with two fp16 multiplicands and f32 compute type exists
    return any(p == 2 for p in prec)


def test_2mm_n8192(torch):
    rng = np.random.default_rng(1)
    samples = {4: _mat_samples(8192, 8192, rng)}
    run(torch, "2mm", [8192], "random", [[1] * 5, [2] * 5, [2, 2, 1, 1, 1]], samples, tc_rel=_tc_chain)


def test_3mm_n8192(torch):
    rng = np.random.default_rng(2)
    samples = {6: _mat_samples(8192, 8192, rng, nr=2, nc=2)}
    run(torch, "3mm", [8192], "random", [[1] * 7, [2, 2, 1, 1, 1, 1, 1]], samples, tc_rel=_tc_chain)


@pytest.mark.parametrize("kind", ["corr", "covar"])
def test_corr_covar_n8192(torch, kind):
    rng = np.random.default_rng(3)
    so = 3 if kind == "corr" else 2
    r = rng.choice(8192, size=48)
    c = rng.choice(8192, size=48)
    samples = {so: (np.concatenate([r, [5]]), np.concatenate([c, [5]]))}
    m = 4 if kind == "corr" else 3
    cfgs = [[1] * m, [0] + [1] * (m - 1)]
    run(torch, kind, [8192, 8192], "random", cfgs, samples)
