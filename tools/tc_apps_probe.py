"""Statement-level tcgen05 rates in the apps: 2MM (plain epilogue) and SYRK/COVAR
(M-major A) at 8192 for f16 / bf16 / E4M3 / E5M2 operands."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

torch.cuda.set_device(0)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
for kind, flops, mk in (("2mm", 4 * N ** 3, lambda t: [t, t, t, t, B.F32]),
                        ("covar", N ** 2 * (N + 1), lambda t: [t, B.F32, B.F32])):
    app = B.App(kind, [N] if kind == "2mm" else [N, N])
    app.set_flags(B.FLAG_FP8)
    ins = gen.make_inputs(kind, app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    for name, t in (("f16", B.F16), ("bf16", B.BF16), ("e4m3", B.E4M3), ("e5m2", B.E5M2)):
        ks = []
        for _ in range(3):
            ks.append(app.run_config(mk(t))["kernel_ms"])
        k = sorted(ks)[1]
        print("%s N=%d %-5s kernel %.3f ms -> %.1f TFLOP/s (statement group, incl. non-TC kernels)" % (
            kind, N, name, k, flops / (k * 1e-3) / 1e12), flush=True)
