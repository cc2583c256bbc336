import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen
torch.cuda.set_device(0)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
app = B.App("conv2d", [N, N])
ins = gen.make_inputs("conv2d", app.objects, "random")
app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
app.reference()
for prec in ([1, 1], [2, 2], [0, 0], [1, 0]):
    for _ in range(2):
        r = app.run_config(prec)
    sa, sb = [{0: 8, 1: 4, 2: 2}[p] for p in prec]
    print(prec, "kernel %.3f ms %.0f GB/s  backconv %.3f ms %.0f GB/s" % (
        r["kernel_ms"], N * N * (sa + sb) / r["kernel_ms"] / 1e6, r["backconv_ms"],
        N * N * (sb + 12) / r["backconv_ms"] / 1e6), flush=True)
