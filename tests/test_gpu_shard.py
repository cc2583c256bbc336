"""Row-sharded fp64 reference (ps_app_reference_rows / ps_app_reference_merge,
SURVEY §8(e)): W shards computed one after another on one GPU, assembled and
merged, are bit-identical to ps_app_reference -- and so are the configuration
results evaluated against them."""
import numpy as np
import pytest

from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import dist as D
from paper_conf_cgo_kangcp20_b200 import inputs as gen

pytestmark = pytest.mark.gpu

CASES = [("gemm", [300, 140, 77], (1.5, 1.2)), ("2mm", [260, 70, 90, 45], None),
         ("3mm", [140, 72, 200, 64, 129], None), ("syrk", [90, 301], (1.5, 1.2)),
         ("syr2k", [66, 259], (1.5, 1.2)), ("corr", [200, 290], None), ("covar", [150, 257], None)]


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


@pytest.mark.parametrize("kind,dims,sc", CASES, ids=[c[0] for c in CASES])
def test_sharded_reference_bit_exact(torch, kind, dims, sc):
    app = B.App(kind, dims, sc)
    ins = gen.make_inputs(kind, app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    full = [r.clone() if r is not None else None for r in app.reference()]
    m = next(k for k, o in enumerate(app.objects) if o["is_output"])
    rows = app.shard_rows
    assert rows == app.objects[m]["rows"] and rows > 0
    assert app.shard_triangular == (kind in ("syrk", "corr", "covar"))
    cols = app.objects[m]["cols"]
    want_res = [app.run_config(app.decode(c)) for c in (0, 1, app.space // 2, app.space - 1)]
    for world in (2, 3, 5):
        b = D.row_bounds(rows, world, app.shard_triangular)
        assembled = app.alloc_refs()
        assembled[m].fill_(float("nan"))
        for r in range(world):
            tmp = app.alloc_refs()
            tmp[m].fill_(float("nan"))
            app.reference_rows(b[r], b[r + 1], tmp)
            assembled[m].view(rows, cols)[b[r]:b[r + 1]] = tmp[m].view(rows, cols)[b[r]:b[r + 1]]
        app.reference_merge(assembled)
        got = assembled[m].cpu().numpy().view(np.uint64)
        assert np.array_equal(got, full[m].cpu().numpy().view(np.uint64)), (kind, world)
        for c, w in zip((0, 1, app.space // 2, app.space - 1), want_res):
            r = app.run_config(app.decode(c))
            assert r["quality"] == w["quality"] and r["max_rel"] == w["max_rel"], (kind, world, c)


def test_not_shardable_and_bad_rows(torch):
    app = B.App("atax", [300, 70])
    ins = gen.make_inputs("atax", app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    assert app.shard_rows == 0
    with pytest.raises(B.PsError):
        app.reference_rows(0, 10, app.alloc_refs())
    g = B.App("gemm", [64])
    gi = gen.make_inputs("gemm", g.objects, "random")
    g.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in gi])
    with pytest.raises(B.PsError):
        g.reference_rows(10, 65, g.alloc_refs())
    with pytest.raises(B.PsError):
        g.reference_rows(5, 4, g.alloc_refs())
    g.reference_rows(7, 7, g.alloc_refs())          # empty shard is fine
