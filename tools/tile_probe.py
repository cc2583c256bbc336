"""Live a3 tile-kernel rates for the mat-vec apps at N=16384: per configuration the
statement-group kernel time (ps_run_config's CUDA events) and the algorithmic GB/s
(one pass over each matrix + vectors), for every A precision crossed with f32/f64
compute types.  One JSON line per configuration, then nvidia-smi clocks.
  python tools/tile_probe.py [app ...]"""
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

torch.cuda.set_device(0)
N = 16384
SZ = {0: 8, 1: 4, 2: 2}
apps = sys.argv[1:] or ["bicg", "atax", "gesummv"]
smi = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks_event_reasons.active",
                        "--format=csv,noheader,nounits", "-lms", "200"], stdout=subprocess.PIPE, text=True)
for kind in apps:
    dims = [N, N] if kind != "gesummv" else [N]
    app = B.App(kind, dims)
    ins = gen.make_inputs(kind, app.objects, "default")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    M = app.num_objects
    for pa in (0, 1, 2):
        for rest in (1, 0):
            prec = [pa] + [rest] * (M - 1)
            if kind == "gesummv":
                prec = [pa, pa] + [rest] * (M - 2)
            app.run_config(prec)
            r = min((app.run_config(prec) for _ in range(5)), key=lambda x: x["kernel_ms"])
            mats = 2 if kind == "gesummv" else 1
            b = mats * N * N * SZ[pa]
            print(json.dumps({"app": kind, "prec": prec, "kernel_ms": round(r["kernel_ms"], 4),
                              "convert_ms": round(r["convert_ms"], 4),
                              "a3_GBps": round(b / (r["kernel_ms"] * 1e-3) / 1e9, 1)}), flush=True)
    del app
    torch.cuda.empty_cache()
smi.terminate()
out, _ = smi.communicate(timeout=10)
sm = [float(l.split(",")[0]) for l in out.strip().splitlines() if l.strip()]
print(json.dumps({"clocks": {"sm_mhz_median": float(np.median(sm)) if sm else None, "samples": len(sm),
                             "reasons": sorted({l.split(",")[1].strip() for l in out.strip().splitlines() if l.strip()})}}))
