"""bench.py's multi-rank entry point on CPU: `--gpus 2 --backend gloo --fake` spawns
two ranks under torch.distributed.run itself, partitions the configuration spaces,
gathers the (fake) result records over gloo and prints one line from rank 0
(VERDICT r1 next #3)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*extra):
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--backend", "gloo", "--fake",
                        "--steps", "2", "--warmup", "3", *extra],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_bench_spawns_two_ranks_gloo():
    line = _run("--gpus", "2")
    assert line["n_gpus"] == 2 and line["fake"] is True
    cfg = line["config"]
    assert cfg["configs_per_step"] == 81 + 243 + 243
    assert len(cfg["configs_per_rank"]) == 2 and sum(cfg["configs_per_rank"]) == 567
    assert min(cfg["configs_per_rank"]) > 0


def test_bench_one_rank_gloo_same_best():
    one = _run("--gpus", "1")
    two = _run("--gpus", "2")
    assert one["n_gpus"] == 1
    assert one["config"]["best_config"] == two["config"]["best_config"]
