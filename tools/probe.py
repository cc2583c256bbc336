"""Quick GPU probe: ps_convert bandwidth per direction, and one app sweep timing."""
import json
import sys
import time

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
from paper_conf_cgo_kangcp20_b200 import binding as B  # noqa: E402
from paper_conf_cgo_kangcp20_b200 import inputs as gen  # noqa: E402

torch.cuda.set_device(0)
SZ = {0: 8, 1: 4, 2: 2}
TD = {0: torch.float64, 1: torch.float32, 2: torch.float16}
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


def time_convert(st, dt, nbytes_src, reps=20):
    n = nbytes_src // SZ[st]
    src = torch.zeros(n, dtype=TD[st], device="cuda")
    dst = torch.empty(n, dtype=TD[dt], device="cuda")
    for _ in range(3):
        B.ps_convert(src, st, dst, dt)
    ts = []
    for _ in range(reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        B.ps_convert(src, st, dst, dt)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    t = float(np.median(ts))
    return n * (SZ[st] + SZ[dt]) / (t * 1e-3) / 1e9, t


out = {}
for st, dt in [(1, 2), (2, 1), (0, 2), (0, 1), (2, 0), (1, 0)]:
    for nb in [1 << 26, 1 << 30, 1 << 32]:
        gbs, t = time_convert(st, dt, nb)
        out["%d->%d@%dMB" % (st, dt, nb >> 20)] = (round(gbs, 1), round(t, 4))
print(json.dumps(out, indent=1))

for kind, dims in [("atax", [16384, 16384]), ("gemm", [64])]:
    app = B.App(kind, dims)
    ins = gen.make_inputs(kind, app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    ids = list(range(app.space))
    app.sweep(ids)
    torch.cuda.synchronize()
    t0 = time.time()
    res, best = app.sweep(ids)
    dt = time.time() - t0
    tot = sum(r["total_ms"] for r in res)
    print(kind, dims, "configs", len(ids), "wall %.3f s -> %.1f configs/s" % (dt, len(ids) / dt),
          "sum total_ms %.2f" % tot, "best", res[best]["config_id"], res[best]["total_ms"],
          "allf32", [r for r in res if r["config_id"] == (3 ** app.num_objects - 1) // 2][0]["total_ms"])
    for r in res[:3] + res[-3:]:
        print("  ", r)
