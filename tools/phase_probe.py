"""Per-app, per-A-precision average phase times of a sweep (diagnostics)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen
torch.cuda.set_device(0)
apps = [("atax", [16384, 16384]), ("bicg", [16384, 16384]), ("gesummv", [16384])]
if len(sys.argv) > 1: apps = [a for a in apps if a[0] in sys.argv[1:]]
for kind, dims in apps:
    app = B.App(kind, dims)
    ins = gen.make_inputs(kind, app.objects, "default")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    ids = list(range(app.space))
    app.sweep_raw(ids)
    arr, _ = app.sweep_raw(ids)
    m = app.num_objects
    pa = arr["config_id"] % 3
    for p in range(3):
        sel = arr[pa == p]
        nbytes = dims[0] * dims[-1] * {0: 8, 1: 4, 2: 2}[p] * (2 if kind == "gesummv" else 1)
        print("%-8s A=%s n=%3d convert %.3f kernel %.3f (%.0f GB/s 1-pass) backconv %.3f total %.3f" % (
            kind, "f64 f32 f16".split()[p], len(sel), sel["convert_ms"].mean(), sel["kernel_ms"].mean(),
            nbytes / (sel["kernel_ms"].mean() * 1e-3) / 1e9, sel["backconv_ms"].mean(), sel["total_ms"].mean()))
