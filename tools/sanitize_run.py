"""Small-shape run of every kernel family, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): conversions with unaligned pointers and ragged n, every app on
ragged dims (tile tails, chunk tails, 2-CTA and 1-CTA tensor-core paths), the quality
kernel, a sweep and a search."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

torch.cuda.set_device(0)
buf = torch.zeros(4096, dtype=torch.uint8, device="cuda")
out = torch.zeros(8192, dtype=torch.uint8, device="cuda")
for st, dt in [(1, 2), (2, 1), (0, 2), (0, 1), (1, 0), (2, 0)]:
    for n in (1, 7, 33, 301):
        for off in (0, 2, 6):
            B.ps_convert(buf.data_ptr() + off * 8, st, out.data_ptr() + off * 8, dt, n)
# the TMA bulk conversion path (>= one 32 KiB chunk per SM) with an unaligned head
# and a ragged remainder, narrowing and widening
big = torch.randint(0, 2 ** 31 - 1, ((1 << 23) // 4 + 1024,), dtype=torch.int32, device="cuda").view(torch.uint8)
bigo = torch.empty(1 << 25, dtype=torch.uint8, device="cuda")
for st, dt in [(1, 2), (2, 0), (0, 1)]:
    n = (1 << 23) // 8 + 37
    B.ps_convert(big.data_ptr() + 8 * 2, st, bigo.data_ptr() + 8 * 2, dt, n)
ref = torch.zeros(301, dtype=torch.float64, device="cuda")
B.ps_quality(torch.zeros(301, device="cuda"), 1, ref)
cases = [("gemm", [70, 130, 33]), ("gemm", [264, 264, 72]), ("2mm", [40, 30, 50, 20]),
         ("3mm", [20, 30, 24, 18, 16]), ("atax", [300, 77]), ("bicg", [270, 93]),
         ("gesummv", [75]), ("corr", [60, 264]), ("covar", [55, 13])]
for kind, dims in cases:
    app = B.App(kind, dims)
    ins = gen.make_inputs(kind, app.objects, "random")
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    ids = list(range(0, app.space, max(1, app.space // 12))) + [app.space - 1]
    app.sweep(ids)
# a row-sharded evaluation (ps_shard_step), two emulated ranks
for kind, dims in [("bicg", [600, 300]), ("corr", [520, 300])]:
    shards = []
    for r in range(2):
        app = B.App(kind, dims)
        ins = gen.make_inputs(kind, app.objects, "random")
        app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
        app.reference()
        shards.append(app)
    prec = [1] * shards[0].num_objects
    stage = 0
    while True:
        outs = [sh.shard_step(prec, r, 2, stage) for r, sh in enumerate(shards)]
        if outs[0][0]:
            break
        for j in range(len(outs[0][1])):
            for q in range(2):
                base, off, ln = outs[q][1][j]
                if ln:
                    shards[1 - q].workspace[base + off:base + off + ln].copy_(
                        shards[q].workspace[base + off:base + off + ln])
        stage += 1
app = B.App("gemm", [64])
ins = gen.make_inputs("gemm", app.objects, "default")
app.bind([torch.from_numpy(a.reshape(-1)).cuda() for a in ins])
app.reference()
app.search(0.9)
torch.cuda.synchronize()
print("sanitize run ok")
