"""Contraction-kernel probe: 2MM statement timings per path (TC / FFMA / DFMA)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen
torch.cuda.set_device(0)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
app = B.App("2mm", [N])
ins = gen.make_inputs("2mm", app.objects, "random")
app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
app.reference()
for name, prec in (("tc f16", [2] * 5), ("simt f32", [1] * 5), ("simt f64", [0] * 5)):
    for _ in range(reps):
        r = app.run_config(prec)
    print("2mm N=%d %-9s kernel %.3f ms -> %.1f TFLOP/s" % (N, name, r["kernel_ms"], 4 * N ** 3 / (r["kernel_ms"] * 1e-3) / 1e12), flush=True)
