"""f64 contraction probe: GEMM / 2MM / CORR statement timings with compute type f64
(the kernel PS_F64_DFMA selects), plus cuBLAS DGEMM (torch.matmul float64) for context."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen
torch.cuda.set_device(0)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
tag = "DFMA" if os.environ.get("PS_F64_DFMA") == "1" else "DMMA"
for kind, flop, precs in (("gemm", 2 * N ** 3, ([0, 0, 0], [1, 1, 0], [2, 2, 0])),
                          ("corr", N ** 2 * (N + 1), ([0, 0, 0, 0], [1, 1, 1, 0])),
                          ("covar", N ** 2 * (N + 1), ([0, 0, 0], [1, 1, 0]))):
    app = B.App(kind, [N])
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
if tag == "DMMA":
    a = torch.randn(N, N, dtype=torch.float64, device="cuda")
    b = torch.randn(N, N, dtype=torch.float64, device="cuda")
    for _ in range(2):
        torch.matmul(a, b)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); torch.matmul(a, b); e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    print("cuBLAS DGEMM N=%d %.3f ms -> %.2f TFLOP/s" % (N, ms, 2 * N ** 3 / (ms * 1e-3) / 1e12))
