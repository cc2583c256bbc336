"""Probe the tcgen05 GEMM: correctness on small shapes vs a torch fp32 matmul of the
fp16 operands (debug aid), and TFLOP/s at 8192^3 (all-f16 2MM statement)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

torch.cuda.set_device(0)
for dims in ([128, 256, 64], [200, 264, 136], [1024, 1024, 1024]):
    app = B.App("gemm", dims, (1.0, 0.0))
    ins = gen.make_inputs("gemm", app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() for a in ins])
    app.reference()
    app.run_config([2, 2, 1])
    got = app.outputs[2].view(dims[0], dims[1]).double()
    a = torch.from_numpy(ins[0]).cuda().half().double().view(dims[0], dims[2])
    b = torch.from_numpy(ins[1]).cuda().half().double().view(dims[2], dims[1])
    want = a @ b
    err = (got - want).abs().max().item()
    print("gemm", dims, "max abs err", err, "max", want.abs().max().item(), flush=True)
    if err > 1e-2 * want.abs().max().item():
        print("  mismatch sample got", got[:2, :8].tolist(), "\n want", want[:2, :8].tolist())
for N in (4096, 8192):
    app = B.App("2mm", [N])
    ins = gen.make_inputs("2mm", app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    for prec in ([2, 2, 2, 2, 2], [2, 2, 1, 2, 1], [1, 1, 1, 1, 1], [0, 0, 0, 0, 0]):
        app.run_config(prec)
        r = app.run_config(prec)
        print("2mm N=%d prec %s kernel %.3f ms -> %.1f TFLOP/s  (q=%.6f)" % (
            N, prec, r["kernel_ms"], 2 * 2 * N ** 3 / (r["kernel_ms"] * 1e-3) / 1e12, r["quality"]), flush=True)
