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
