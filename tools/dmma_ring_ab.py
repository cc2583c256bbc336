"""DMMA statement rates (f64 / f32 / f16 operands into f64 statements) at 8192^3 for an A/B of
library builds (profiles/dmma_ab_*_r2ay.jsonl)."""
import json, sys, os
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen
N = 8192
torch.cuda.set_device(0)
for prec in ([0, 0, 0], [1, 1, 0], [2, 1, 0]):
    app = B.App("gemm", [N])
    ins = gen.make_inputs("gemm", app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    app.run_config(prec)
    ms = min(app.run_config(prec)["kernel_ms"] for _ in range(4))
    print(json.dumps({"prec": prec, "kernel_ms": round(ms, 3), "tflops": round(2.0 * N ** 3 / (ms * 1e-3) / 1e12, 2)}), flush=True)
    del app
    torch.cuda.empty_cache()
