"""Row-sharded evaluation of ONE configuration (prescaler.h (4b), SURVEY §8(e) "very
large objects: contiguous row-range shards"), emulated on one GPU: W apps share
the inputs, each runs its stages of ps_shard_step, and after every stage each
shard's produced byte ranges are copied into the other shards' workspaces (what
an NCCL all-gather does across GPUs, dist.exchange_regions).  The records and the
delivered outputs must be bit-identical to the unsharded ps_run_config for
W = 2, 3, 5 (including empty shards), in f64 / f32 / f16 (tcgen05) / mixed
configurations, for all 14 apps (FDTD-2D exchanging one halo row of ey and of hz
per time step)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

CASES = {
    "atax": [1100, 900], "bicg": [1100, 900], "gesummv": [1100], "mvt": [1100],
    "gemm": [1100, 300, 200], "2mm": [1100, 260, 200, 300], "3mm": [1100, 600, 200, 300, 250],
    "syr2k": [300, 1100], "syrk": [300, 1100], "corr": [1000, 1100], "covar": [1000, 1100],
    "conv2d": [1100, 700], "conv3d": [40, 30, 50], "fdtd2d": [5, 600, 300],
}


def _configs(app, k=3):
    M = app.num_objects
    ids = {0, (3 ** M - 1) // 2, 3 ** M - 1}
    rng = np.random.default_rng(len(app.kind) * 7 + M)
    while len(ids) < 3 + k:
        ids.add(int(rng.integers(0, 3 ** M)))
    return sorted(ids)


def _run_sharded(torch, shards, prec, W):
    stage = 0
    while True:
        outs = [sh.shard_step(prec, r, W, stage) for r, sh in enumerate(shards)]
        dones = {o[0] for o in outs}
        assert len(dones) == 1, "ranks disagree on the stage count"
        if outs[0][0]:
            return [o[2] for o in outs]
        nreg = {len(o[1]) for o in outs}
        assert len(nreg) == 1
        for j in range(nreg.pop()):
            for q, (_, regs, _) in enumerate(outs):
                base, off, ln = regs[j]
                if not ln:
                    continue
                src = shards[q].workspace[base + off:base + off + ln]
                for t, sh in enumerate(shards):
                    if t != q:
                        b2, _, _ = outs[t][1][j]
                        assert b2 == base            # same layout on every rank
                        sh.workspace[base + off:base + off + ln].copy_(src)
        torch.cuda.synchronize()
        stage += 1


@pytest.mark.parametrize("kind", sorted(CASES))
def test_sharded_equals_unsharded(kind):
    import torch
    from paper_conf_cgo_kangcp20_b200 import binding as B
    from paper_conf_cgo_kangcp20_b200 import inputs as gen
    dims = CASES[kind]
    base = B.App(kind, dims)
    ins = gen.make_inputs(kind, base.objects, "random", seed=5)
    dins = [torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins]
    base.bind(dins)
    refs = base.reference()
    assert base.eval_shard_rows > 0
    outm = [m for m, o in enumerate(base.objects) if o["is_output"]]
    for cid in _configs(base):
        prec = base.decode(cid)
        want = base.run_config(prec)
        want_out = {m: base.outputs[m].clone() for m in outm}
        for W in (2, 3, 5):
            shards = []
            for _ in range(W):
                sh = B.App(kind, dims)
                sh.bind(dins)
                sh.set_reference(refs)
                for m in outm:
                    sh.outputs[m].fill_(float("nan"))
                shards.append(sh)
            got = _run_sharded(torch, shards, prec, W)
            for r, g in enumerate(got):
                for k in ("config_id", "quality", "max_rel", "nonfinite", "pass"):
                    assert g[k] == want[k], (kind, cid, W, r, k, g[k], want[k])
            rows_total = base.eval_shard_rows
            for m in outm:
                o = base.objects[m]
                w = want_out[m].view(o["rows"], o["cols"])
                for r, sh in enumerate(shards):
                    g = sh.outputs[m].view(o["rows"], o["cols"])
                    if o["rows"] == 1:                                   # vector outputs: whole
                        assert torch.equal(g.view(torch.int32), w.view(torch.int32)), (kind, cid, W, r, m)
                    else:
                        r0, r1 = sh.shard_bounds(r, W)
                        assert o["rows"] == rows_total
                        assert torch.equal(g[r0:r1].contiguous().view(torch.int32),
                                           w[r0:r1].contiguous().view(torch.int32)), (kind, cid, W, r, m)
            del shards


def test_bounds_cover_and_align():
    from paper_conf_cgo_kangcp20_b200 import binding as B
    for kind, dims in CASES.items():
        app = B.App(kind, dims)
        rows = app.eval_shard_rows
        for W in (1, 2, 3, 5, 8):
            b = [app.shard_bounds(r, W) for r in range(W)]
            assert b[0][0] == 0 and b[-1][1] == rows
            for (a0, a1), (c0, c1) in zip(b, b[1:]):
                assert a1 == c0 and a0 <= a1


def test_fp8_objects_are_rejected():
    """A per-tensor fp8 scale needs the amax of the whole object: not row-shardable."""
    import torch
    from paper_conf_cgo_kangcp20_b200 import binding as B
    from paper_conf_cgo_kangcp20_b200 import inputs as gen
    app = B.App("gemm", [300, 200, 100])
    app.set_flags(B.FLAG_FP8)
    ins = gen.make_inputs("gemm", app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() for a in ins])
    app.reference()
    with pytest.raises(B.PsError):
        app.shard_step([4, 4, 1], 0, 2, 0)
