"""tcgen05 throughput probe: GEMM C = A.B at N^3 with A, B in fp16 / bf16 / E4M3 /
E5M2 (C f32), kernel_ms from the library's CUDA events -> TFLOP/s; also the a2
conversion time of the two operands (fp8: amax + encode)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

torch.cuda.set_device(0)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
app = B.App("gemm", [N], (1.0, 0.0))
app.set_flags(B.FLAG_FP8)
ins = gen.make_inputs("gemm", app.objects, "random")
app.bind([torch.from_numpy(a.reshape(-1)).cuda() for a in ins])
app.reference()
for name, prec in (("f16", [B.F16, B.F16, B.F32]), ("bf16", [B.BF16, B.BF16, B.F32]),
                   ("e4m3", [B.E4M3, B.E4M3, B.F32]), ("e5m2", [B.E5M2, B.E5M2, B.F32]),
                   ("e4m3 x e5m2", [B.E4M3, B.E5M2, B.F32])):
    ks, cs = [], []
    for _ in range(reps):
        r = app.run_config(prec)
        ks.append(r["kernel_ms"])
        cs.append(r["convert_ms"])
    k = sorted(ks)[len(ks) // 2]
    c = sorted(cs)[len(cs) // 2]
    print("gemm N=%d %-12s kernel %.3f ms -> %.1f TFLOP/s   convert %.3f ms   q=%.6f" % (
        N, name, k, 2 * N ** 3 / (k * 1e-3) / 1e12, c, r["quality"]), flush=True)
