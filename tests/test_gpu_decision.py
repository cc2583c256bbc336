"""System Inspector (ps_transfer DB), Alg. 2 method choice and the whole-program
Decision Maker (Alg. 1 with PFP and the wildcard test) on the GPU."""
import numpy as np
import pytest

from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import decision as D
from paper_conf_cgo_kangcp20_b200 import inputs as gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


@pytest.fixture(scope="module")
def db(torch):
    return D.inspect(sizes=(1 << 18, 1 << 22, 1 << 24), reps=3)


def test_inspector_db(db):
    assert len(db["entries"]) == 3 * 3 * 5
    for e in db["entries"]:
        assert e["ms"] > 0
    # which method wins is what the inspector measures (system-dependent);
    # Alg. 2 must return the minimum of the candidates it is given
    n = 1 << 24
    for dt in (B.F64, B.F32, B.F16):
        m, inter, t = D.best_method(db, n, dt)
        assert t == min(D.expected_ms(db, k, dt, n) for k in D.DIRECT)
        print("n=2^24 dst=%d: %s" % (dt, {D.NAMES[k]: round(D.expected_ms(db, k, dt, n), 3)
                                          for k in D.METHODS}))


def test_ps_transfer_values(torch):
    x = (torch.rand(100003) * 7e4).float()
    h = x.pin_memory()
    stage = torch.empty(100003 * 4, dtype=torch.uint8, device="cuda")
    want = {}
    for dt in (B.F64, B.F32, B.F16):
        outs = []
        for meth in D.DIRECT:
            dst = torch.empty(100003 * 8, dtype=torch.uint8, device="cuda")
            B.ps_transfer(h, dst, dt, 100003, meth, 4, stage)
            outs.append(dst[:100003 * D.SIZE[dt]].cpu().numpy())
        for o in outs[1:]:
            assert np.array_equal(o, outs[0]), dt


@pytest.mark.parametrize("kind,dims,iset", [("bicg", [4096, 4096], "default"),
                                            ("gemm", [512], "random"),
                                            ("atax", [2048, 2048], "random")])
def test_decision_maker(torch, db, kind, dims, iset):
    app = B.App(kind, dims)
    ins = gen.make_inputs(kind, app.objects, iset)
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    host = [torch.from_numpy(a.reshape(-1)).pin_memory() if a is not None else None for a in ins]
    res = D.decide(app, host, db, toq=0.9)
    m = app.num_objects
    assert res["result"]["pass"]
    # PFP (3) + per object at most 2 types + one wildcard verification  (Eq. 3)
    assert res["trials"] <= 3 + 3 * m
    assert res["trials"] < res["space"] * 5
    # the original program: every object f32, transferred as f32
    orig = app.run_config_host([B.F32] * m, host, [B.XFER_DEVICE] * m)
    print("%s: chosen %s %s %.3f ms vs original %.3f ms (%d trials)" % (
        kind, res["prec"], res["method_names"], res["result"]["total_ms"], orig["total_ms"],
        res["trials"]))
