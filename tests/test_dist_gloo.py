"""Multi-process (world_size 2, gloo, CPU) tests of the multi-GPU sweep logic:
deterministic LPT partition, result gather, identical best config on every rank."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import dist as D


def test_partition_covers_every_config_once():
    objs = oracle.app_objects("corr", [8192, 8192])
    ids = list(range(81))
    for world in (1, 2, 3, 4, 8):
        parts = [D.partition_configs("corr", [8192, 8192], objs, ids, world, r) for r in range(world)]
        flat = sorted(c for p in parts for c in p)
        assert flat == ids
        costs = {c: D.config_cost("corr", [8192, 8192], objs, c) for c in ids}
        loads = [sum(costs[c] for c in p) for p in parts]
        # LPT bound: makespan <= 4/3 OPT, OPT >= max(total/world, max cost)
        opt_lb = max(sum(costs.values()) / world, max(costs.values()))
        assert max(loads) <= 4.0 / 3.0 * opt_lb + 1e-12


def test_cost_model_orders_precisions():
    objs = oracle.app_objects("2mm", [8192])
    c64 = D.config_cost("2mm", [8192], objs, 0)
    c32 = D.config_cost("2mm", [8192], objs, (3 ** 5 - 1) // 2)
    c16 = D.config_cost("2mm", [8192], objs, 3 ** 5 - 1)
    assert c64 > c32 > c16


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _fake_eval(kind, dims, cid):
    """Deterministic stand-in for ps_sweep records (no GPU)."""
    rec = np.zeros(1, dtype=B.RESULT_DTYPE)
    rng = np.random.default_rng(cid)
    rec["config_id"] = cid
    rec["total_ms"] = np.float32(1.0 + (cid * 7919 % 13))
    rec["quality"] = 1.0 - rng.random() * 0.2
    rec["pass"] = int(rec["quality"][0] >= 0.9)
    return rec


def _worker(rank, world, port, kind, dims, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    objs = oracle.app_objects(kind, dims)
    ids = list(range(3 ** len(objs)))
    mine = D.partition_configs(kind, dims, objs, ids, world, rank)
    local = np.concatenate([_fake_eval(kind, dims, c) for c in mine]) if mine else \
        np.zeros(0, dtype=B.RESULT_DTYPE)
    full = D.gather_results(local)
    q.put((rank, full.tobytes(), D.best_index(full), len(mine)))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gather_world2_gloo(world):
    kind, dims = "bicg", [16384, 16384]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, kind, dims, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    out.sort()
    tables = [np.frombuffer(o[1], dtype=B.RESULT_DTYPE) for o in out]
    expect = np.concatenate([_fake_eval(kind, dims, c) for c in range(243)])
    for t in tables:
        assert t.tobytes() == expect.tobytes()
    assert len({o[2] for o in out}) == 1
    assert out[0][2] == D.best_index(expect)
    assert sum(o[3] for o in out) == 243 and min(o[3] for o in out) > 0


# ------------------------------------------------------------ sharded reference
@pytest.mark.parametrize("triangular", [False, True])
def test_row_bounds_cover_and_balance(triangular):
    for rows in (1, 7, 100, 8192):
        for world in (1, 2, 3, 8):
            b = D.row_bounds(rows, world, triangular)
            assert len(b) == world + 1 and b[0] == 0 and b[-1] == rows
            assert all(b[r] <= b[r + 1] for r in range(world))
            cost = (lambda i: rows - i) if triangular else (lambda i: 1)
            loads = [sum(cost(i) for i in range(b[r], b[r + 1])) for r in range(world)]
            total = sum(loads)
            assert max(loads) <= total / world + cost(0) + 1e-9


def _rows_worker(rank, world, port, kind, dims, q):
    """Each rank holds only its rows of the oracle's fp64 reference (the rest NaN, the
    strictly-lower part of triangular outputs garbage, as ps_app_reference_rows leaves
    them); gather_rows must reassemble every row on every rank."""
    import torch
    import torch.distributed as dist
    from paper_conf_cgo_kangcp20_b200 import inputs as gen
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    objs = oracle.app_objects(kind, dims)
    ins = gen.make_inputs(kind, objs, "random")
    ref = oracle.reference(kind, dims, ins)
    m = next(k for k, o in enumerate(objs) if o["is_output"])
    rows, cols = objs[m]["rows"], objs[m]["cols"]
    tri = kind in ("syrk", "corr", "covar")
    b = D.row_bounds(rows, world, tri)
    mine = np.full((rows, cols), np.nan)
    want = ref[m].reshape(rows, cols)
    mine[b[rank]:b[rank + 1]] = want[b[rank]:b[rank + 1]]
    full = torch.from_numpy(mine.reshape(-1).copy())
    D.gather_rows(full, b, rank, cols)
    q.put((rank, full.numpy().tobytes()))
    dist.destroy_process_group()


@pytest.mark.parametrize("kind,dims", [("corr", [37, 29]), ("2mm", [21, 17, 13, 11])])
def test_gather_rows_world2_gloo(kind, dims):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rows_worker, args=(r, 2, port, kind, dims, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    from paper_conf_cgo_kangcp20_b200 import inputs as gen
    objs = oracle.app_objects(kind, dims)
    ref = oracle.reference(kind, dims, gen.make_inputs(kind, objs, "random"))
    m = next(k for k, o in enumerate(objs) if o["is_output"])
    for _, raw in out:
        got = np.frombuffer(raw, dtype=np.float64)
        assert got.tobytes() == np.ascontiguousarray(ref[m], dtype=np.float64).reshape(-1).tobytes()


# ------------------------------------------- row-sharded evaluation exchange
def _xchg_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ws = torch.zeros(4096, dtype=torch.uint8)
    # two regions at workspace offsets 100 and 2000; rank r owns uneven (possibly empty) ranges
    spans = [[(0, 37), (37, 37), (37, 300)], [(0, 8), (8, 24), (24, 1000)]]
    regions = []
    for j, base in enumerate((100, 2000)):
        o0, o1 = spans[j][rank]
        ws[base + o0:base + o1] = torch.arange(o0, o1, dtype=torch.int64).to(torch.uint8) + 7 * j + 1
        regions.append((base, o0, o1 - o0))
    D.exchange_regions(ws, regions)
    q.put((rank, ws.numpy().tobytes()))
    dist.destroy_process_group()


def test_exchange_regions_world3_gloo():
    """dist.exchange_regions (the NCCL all-gather of ps_shard_step's byte ranges):
    every rank ends with every rank's range, including empty ones."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_xchg_worker, args=(r, 3, port, q)) for r in range(3)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=120) for _ in range(3))
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    want = np.zeros(4096, dtype=np.uint8)
    want[100:400] = (np.arange(300) + 1).astype(np.uint8)
    want[2000:3000] = (np.arange(1000) + 8).astype(np.uint8)
    for _, raw in out:
        assert np.frombuffer(raw, dtype=np.uint8).tobytes() == want.tobytes()


@pytest.mark.parametrize("radix", [4, 6])
def test_partition_bf16_fp8_spaces(radix):
    """the cost model covers the bf16 (radix 4) and fp8 (radix 6) alphabets --
    fp8 objects are 1 byte and fp8 x fp8 contractions are costed on tcgen05 f8f6f4."""
    objs = oracle.app_objects("2mm", [512])
    ids = list(range(radix ** len(objs)))
    parts = [D.partition_configs("2mm", [512], objs, ids, 3, r, radix=radix) for r in range(3)]
    assert sorted(c for p in parts for c in p) == ids
    if radix == 6:
        e4 = D.config_cost("2mm", [512], objs, sum(4 * 6 ** m for m in range(5)), 6)
        f16 = D.config_cost("2mm", [512], objs, sum(2 * 6 ** m for m in range(5)), 6)
        assert e4 < f16      # fp8 moves half the bytes and runs at twice the tensor rate
