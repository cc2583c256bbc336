"""f32 contraction probe: GEMM / 2MM / CORR statement timings with compute type f32
(gemm_ffma.cu, or the previous kernel with PS_F32_SIMT_OLD=1)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen
torch.cuda.set_device(0)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
tag = "old" if os.environ.get("PS_F32_SIMT_OLD") == "1" else "ffma"
for kind, flop, precs in (("gemm", 2 * N ** 3, ([1, 1, 1], [2, 1, 1], [1, 2, 1])),
                          ("corr", N ** 2 * (N + 1), ([1, 1, 1, 1], [1, 1, 1, 2])),
                          ("covar", N ** 2 * (N + 1), ([1, 1, 1],))):
    app = B.App(kind, [N])
    app.set_flags(B.FLAG_NO_TENSOR_CORES)
    ins = gen.make_inputs(kind, app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    for prec in precs:
        best = 1e9
        for _ in range(3):
            r = app.run_config(prec)
            best = min(best, r["kernel_ms"])
        print("%s %-5s N=%d prec %s kernel %.3f ms -> %.2f TFLOP/s (statement group)" % (
            tag, kind, N, prec, best, flop / (best * 1e-3) / 1e12), flush=True)
    del app
