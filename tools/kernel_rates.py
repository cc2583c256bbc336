"""Contraction kernel rates at N^3 (default 8192) with a clock record: the library's
statement kernels through ps_run_config (CUDA events on the launching stream, best
of 5 after warm-up) next to cuBLAS on the same box, plus nvidia-smi clocks sampled
during the run.  One JSON line per measurement, a final clocks line.

  python tools/kernel_rates.py [N] [which,...]   which in {f32,f64,tc,cublas}"""
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
WHICH = set((sys.argv[2] if len(sys.argv) > 2 else "f32,f64,tc,cublas").split(","))
torch.cuda.set_device(0)
smi = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active",
                        "--format=csv,noheader,nounits", "-lms", "200"], stdout=subprocess.PIPE, text=True)


def emit(**kw):
    print(json.dumps(kw), flush=True)


def lib_rate(kind, prec, flags, flop, label, reps=5):
    app = B.App(kind, [N])
    app.set_flags(flags)
    ins = gen.make_inputs(kind, app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    app.run_config(prec)
    ms = min(app.run_config(prec)["kernel_ms"] for _ in range(reps))
    emit(kernel=label, app=kind, N=N, prec=prec, kernel_ms=round(ms, 4), tflops=round(flop / (ms * 1e-3) / 1e12, 1))
    del app
    torch.cuda.empty_cache()


gemm = 2.0 * N ** 3
if "f32" in WHICH:   # FFMA (SIMT, R3-exact): GEMM all-f32 (A k-major), f16 A, f16 B
    for prec in ([1, 1, 1], [2, 1, 1], [1, 2, 1]):
        lib_rate("gemm", prec, B.FLAG_NO_TENSOR_CORES, gemm, "gemm_ffma_kernel")
if "f64" in WHICH:   # DMMA chains
    lib_rate("gemm", [0, 0, 0], 0, gemm, "gemm_dmma_kernel")
if "tcplain" in WHICH:   # C = A.B written plainly (no alpha/beta read of C): 2MM with every object
    # f16 but E, NL = 256 -- both statements on tcgen05, the second 3% of the flops
    def lib_rate_dims(kind, dims, prec, flags, flop, label, reps=5):
        app = B.App(kind, dims)
        app.set_flags(flags)
        ins = gen.make_inputs(kind, app.objects, "random")
        app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
        app.reference()
        app.run_config(prec)
        ms = min(app.run_config(prec)["kernel_ms"] for _ in range(reps))
        emit(kernel=label, app=kind, dims=dims, prec=prec, kernel_ms=round(ms, 4),
             tflops=round(flop / (ms * 1e-3) / 1e12, 1))
        del app
        torch.cuda.empty_cache()
    d = [N, N, N, 256]
    fl = 2.0 * N ** 3 + 2.0 * N * N * 256
    lib_rate_dims("2mm", d, [2, 2, 2, 2, 1], 0, fl, "gemm_tc2_kernel fp16, plain epilogue (C f16, then E = C.D, NL 256)")
    lib_rate_dims("2mm", d, [3, 3, 3, 3, 1], B.FLAG_BF16, fl, "gemm_tc2_kernel bf16, plain epilogue (C bf16, then E = C.D, NL 256)")
if "tc" in WHICH:    # tcgen05: fp16, bf16, e4m3, e5m2 multiplicands, f32 C
    lib_rate("gemm", [2, 2, 1], 0, gemm, "gemm_tc2_kernel fp16")
    lib_rate("gemm", [3, 3, 1], B.FLAG_BF16, gemm, "gemm_tc2_kernel bf16")
    lib_rate("gemm", [4, 4, 1], B.FLAG_FP8, gemm, "gemm_tc2_kernel e4m3")
    lib_rate("gemm", [5, 5, 1], B.FLAG_FP8, gemm, "gemm_tc2_kernel e5m2")
if "tcaxpby" in WHICH:   # alpha/beta GEMM with a 16-bit C (Cin read + C write in fp16 / bf16),
    # the same operation as cuBLAS addmm(beta, C, alpha, A, B) below
    lib_rate("gemm", [2, 2, 2], 0, gemm, "gemm_tc2_kernel fp16, alpha/beta epilogue, C fp16")
    lib_rate("gemm", [3, 3, 3], B.FLAG_BF16, gemm, "gemm_tc2_kernel bf16, alpha/beta epilogue, C bf16")
if "cublas" in WHICH:
    def tm(f, reps=10):
        f()
        torch.cuda.synchronize()
        best = 1e9
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            f()
            e1.record()
            torch.cuda.synchronize()
            best = min(best, e0.elapsed_time(e1))
        return best
    for dt in (torch.float16, torch.bfloat16, torch.float64):
        a = torch.randn(N, N, device="cuda").to(dt)
        b = torch.randn(N, N, device="cuda").to(dt)
        ms = tm(lambda: a @ b)
        emit(kernel="cuBLAS matmul", dtype=str(dt), N=N, kernel_ms=round(ms, 4), tflops=round(gemm / (ms * 1e-3) / 1e12, 1))
        del a, b
    for dt in (torch.float16, torch.bfloat16):   # C <- beta C + alpha A B, 16-bit C read and written
        a = torch.randn(N, N, device="cuda").to(dt)
        b = torch.randn(N, N, device="cuda").to(dt)
        c = torch.randn(N, N, device="cuda").to(dt)
        ms = tm(lambda: torch.addmm(c, a, b, beta=0.5, alpha=1.5))
        emit(kernel="cuBLAS addmm (beta C + alpha A B)", dtype=str(dt), N=N, kernel_ms=round(ms, 4),
             tflops=round(gemm / (ms * 1e-3) / 1e12, 1))
        del a, b, c
    # f32 with TF32 off: cuBLAS's own FFMA SGEMM, the practical ceiling for gemm_ffma_kernel
    torch.backends.cuda.matmul.allow_tf32 = False
    a = torch.randn(N, N, device="cuda")
    b = torch.randn(N, N, device="cuda")
    ms = tm(lambda: a @ b, reps=3)
    emit(kernel="cuBLAS matmul (FFMA, tf32 off)", dtype="torch.float32", N=N, kernel_ms=round(ms, 4),
         tflops=round(gemm / (ms * 1e-3) / 1e12, 1))
    del a, b
    try:
        a = torch.randn(N, N, device="cuda").to(torch.float8_e4m3fn)
        b = torch.randn(N, N, device="cuda").to(torch.float8_e4m3fn).t()
        one = torch.ones((), device="cuda")
        ms = tm(lambda: torch._scaled_mm(a, b, scale_a=one, scale_b=one, out_dtype=torch.float32))
        emit(kernel="cuBLAS _scaled_mm", dtype="e4m3", N=N, kernel_ms=round(ms, 4), tflops=round(gemm / (ms * 1e-3) / 1e12, 1))
    except Exception as e:   # pragma: no cover
        emit(kernel="cuBLAS _scaled_mm", error=str(e)[:200])

smi.terminate()
out, _ = smi.communicate(timeout=10)
sm = [float(l.split(",")[0]) for l in out.strip().splitlines() if l.strip()]
reasons = sorted({l.split(",")[3].strip() for l in out.strip().splitlines() if l.strip()})
emit(clocks={"sm_mhz_median": float(np.median(sm)) if sm else None, "sm_mhz_max": max(sm) if sm else None,
             "samples": len(sm), "active_reason_masks": reasons})
