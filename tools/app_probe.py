"""Per-configuration phase times of one app (tool; not part of the product path).
usage: python tools/app_probe.py KIND D0,D1,.. [cid,cid,..|all] [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cgo_kangcp20_b200 import binding as B  # noqa: E402
from paper_conf_cgo_kangcp20_b200 import inputs as gen  # noqa: E402

kind = sys.argv[1]
dims = [int(x) for x in sys.argv[2].split(",")]
torch.cuda.set_device(0)
app = B.App(kind, dims)
ins = gen.make_inputs(kind, app.objects, "random")
app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
app.reference()
sel = sys.argv[3] if len(sys.argv) > 3 else "all"
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 2
ids = range(app.space) if sel == "all" else [int(x) for x in sel.split(",")]
for cid in ids:
    prec = app.decode(cid)
    for _ in range(reps):
        r = app.run_config(prec)
    print("%4d %s convert %.3f kernel %.3f backconv %.3f quality %.3f ms  Q=%.6f" % (
        cid, prec, r["convert_ms"], r["kernel_ms"], r["backconv_ms"], r["quality_ms"], r["quality"]),
        flush=True)
