"""Reference rates on this box for the tcgen05 comparison (library GEMMs, context
only): torch.matmul fp16/bf16 (cuBLAS) and torch._scaled_mm fp8 at N^3, timed with
CUDA events after warm-up; plus our kernel's 1-SM variant when PS_TC_1SM is set."""
import sys
import torch

N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
reps = 10
a = torch.randn(N, N, device="cuda")
b = torch.randn(N, N, device="cuda")


def timeit(f):
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(reps):
        e0.record()
        f()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2]


for dt in (torch.float16, torch.bfloat16):
    x, y = a.to(dt), b.to(dt)
    t = timeit(lambda: torch.matmul(x, y))
    print("cublas %-9s %.3f ms -> %.1f TFLOP/s" % (str(dt).split(".")[1], t, 2 * N ** 3 / t / 1e9), flush=True)
try:
    x = a.to(torch.float8_e4m3fn)
    y = b.to(torch.float8_e4m3fn).t().contiguous().t()
    one = torch.ones((), device="cuda")
    t = timeit(lambda: torch._scaled_mm(x, y, scale_a=one, scale_b=one, out_dtype=torch.float32))
    print("cublas e4m3      %.3f ms -> %.1f TFLOP/s" % (t, 2 * N ** 3 / t / 1e9), flush=True)
except Exception as e:  # pragma: no cover
    print("scaled_mm unavailable:", e)
