"""Whole-program evaluation from host inputs (ps_run_config_host) with every
type-conversion method of Fig. 3.

Methods (a) single loop, (b) multithreaded SIMD, (c) device, (e) pipelined deliver
exactly the objects the device-resident path builds -> bit-identical outputs and
quality.  (d) transient conversion through fp16 equals the oracle run on inputs
rounded through fp16 ("transient conversion can incur more errors").
"""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

pytestmark = pytest.mark.gpu
METHODS = [B.XFER_DEVICE, B.XFER_HOST_LOOP, B.XFER_HOST_SIMD, B.XFER_PIPELINE]


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def make(torch, kind, dims, iset):
    app = B.App(kind, dims)
    app.set_flags(B.FLAG_NO_TENSOR_CORES)
    ins = gen.make_inputs(kind, app.objects, iset)
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    host = [torch.from_numpy(a.reshape(-1)).pin_memory() if a is not None else None for a in ins]
    return app, ins, host


@pytest.mark.parametrize("kind,dims", [("gemm", [200, 150, 70]), ("bicg", [5000, 4100]),
                                       ("corr", [300, 70]), ("gesummv", [3001])])
def test_methods_match_device_path(torch, kind, dims):
    app, ins, host = make(torch, kind, dims, "random")
    rng = np.random.default_rng(1)
    outs = [torch.empty(o["n"], dtype=torch.float32).pin_memory() if o["is_output"] else None
            for o in app.objects]
    for cid in [0, (3 ** app.num_objects - 1) // 2, 3 ** app.num_objects - 1] + \
            list(rng.integers(0, app.space, 4)):
        prec = app.decode(int(cid))
        ref = app.run_config(prec)
        dev_out = [t.cpu().numpy().copy() if t is not None else None for t in app.outputs]
        for meth in METHODS:
            methods = [meth] * app.num_objects
            r = app.run_config_host(prec, host, methods, host_outputs=outs, threads=4)
            assert r["quality"] == ref["quality"] and r["max_rel"] == ref["max_rel"], (prec, meth)
            assert r["nonfinite"] == ref["nonfinite"]
            assert r["transfer_ms"] > 0 and r["total_ms"] >= r["transfer_ms"]
            for m, o in enumerate(app.objects):
                if o["is_output"]:
                    a, b = outs[m].numpy(), dev_out[m]
                    assert np.array_equal(a.view(np.uint32), b.view(np.uint32)) or \
                        np.array_equal(np.isnan(a), np.isnan(b)), (prec, meth, m)


@pytest.mark.parametrize("kind,dims", [("gemm", [130, 70, 90]), ("atax", [600, 336])])
def test_transient_equals_oracle_on_fp16_rounded_inputs(torch, kind, dims):
    app, ins, host = make(torch, kind, dims, "random")
    oref = oracle.reference(kind, dims, ins)
    for cid in [0, (3 ** app.num_objects - 1) // 2, 5]:
        prec = app.decode(cid)
        methods = [B.XFER_TRANSIENT] * app.num_objects
        r = app.run_config_host(prec, host, methods)
        # transient inputs: f32 -> f16 on the host, f16 -> c(m) on the device
        tins = [None if a is None else oracle.convert(oracle.convert(a.reshape(-1), 1, 2), 2, 1)
                for a in ins]
        ro, delivered = oracle.evaluate(kind, dims, prec, tins, oref)
        assert abs(r["quality"] - ro["quality"]) <= 1e-12 and r["max_rel"] == ro["max_rel"], prec
        for m, o in enumerate(app.objects):
            if o["is_output"]:
                got = app.outputs[m].cpu().numpy()
                assert np.array_equal(got.view(np.uint32), delivered[m].reshape(-1).view(np.uint32))


def test_mixed_methods_per_object(torch):
    app, ins, host = make(torch, "gesummv", [2048], "default")
    prec = [B.F16, B.F32, B.F16, B.F32, B.F64]
    base = app.run_config(prec)
    r = app.run_config_host(prec, host, [B.XFER_PIPELINE, B.XFER_HOST_SIMD, B.XFER_DEVICE,
                                         B.XFER_DEVICE, B.XFER_DEVICE])
    assert r["quality"] == base["quality"]
