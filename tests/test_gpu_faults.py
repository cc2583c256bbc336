"""Fault injection: NaN, +-inf, subnormal and fp16-overflowing values in
the inputs flow through every configuration exactly as the oracle says (NaN-aware
bit-exact delivered outputs, identical non-finite counts and max error)."""
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


def poison(a, rng):
    a = a.copy().reshape(-1)
    idx = rng.choice(a.size, size=min(a.size, 40), replace=False)
    vals = np.array([np.nan, np.inf, -np.inf, 1e-40, -3e-42, 7e4, -9e4, 2.0 ** -24, 2.0 ** -25, 65520.0],
                    dtype=np.float32)
    a[idx] = vals[np.arange(idx.size) % vals.size]
    return a


@pytest.mark.parametrize("kind,dims", [("gemm", [70, 66, 33]), ("bicg", [300, 257]),
                                       ("gesummv", [301]), ("covar", [130, 37])])
def test_poisoned_inputs(torch, kind, dims):
    rng = np.random.default_rng(9)
    app = B.App(kind, dims)
    app.set_flags(B.FLAG_NO_TENSOR_CORES)
    ins = [None if a is None else poison(a, rng).reshape(a.shape)
           for a in gen.make_inputs(kind, app.objects, "random")]
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    oref = oracle.reference(kind, dims, ins)
    for cid in range(0, app.space, max(1, app.space // 27)):
        prec = app.decode(cid)
        r = app.run_config(prec)
        ro, delivered = oracle.evaluate(kind, dims, prec, ins, oref)
        assert r["nonfinite"] == ro["nonfinite"], prec
        assert (r["max_rel"] == ro["max_rel"]) or (np.isnan(r["max_rel"]) and np.isnan(ro["max_rel"]))
        assert abs(r["quality"] - ro["quality"]) <= 1e-12
        for m, o in enumerate(app.objects):
            if o["is_output"]:
                got = app.outputs[m].cpu().numpy()
                want = delivered[m].reshape(-1)
                same = (got.view(np.uint32) == want.view(np.uint32)) | (np.isnan(got) & np.isnan(want))
                assert np.all(same), (prec, m, np.flatnonzero(~same)[:5])
