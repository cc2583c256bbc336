"""Run under ncu to measure DRAM bytes per launch of the a2 conversion kernel in each
direction of the headline mix (and the other sweep directions), on 1 GiB of random
bit patterns, one launch per direction after one warm-up launch:

  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
      --clock-control none -k regex:convert --csv --log-file gpurun_out/traffic.csv \
      python tools/traffic_probe.py
  python tools/traffic_probe.py --summarise gpurun_out/traffic.csv profiles/ncu_traffic_convert_r2.json

Launch order = DIRECTIONS x (warm-up, measured); the summary keeps the measured one."""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
DIRECTIONS = [(1, 2, "f32->f16"), (1, 0, "f32->f64"), (2, 1, "f16->f32"), (0, 2, "f64->f16"),
              (0, 1, "f64->f32"), (1, 3, "f32->bf16"), (1, 1, "f32->f32 copy")]
KERNEL_DIRECTIONS = [d for d in DIRECTIONS if d[0] != d[1]]   # same type: cudaMemcpyAsync, no kernel
SZ = {0: 8, 1: 4, 2: 2, 3: 2}
SRC_BYTES = 1 << 30


def run():
    import torch
    from paper_conf_cgo_kangcp20_b200 import binding as B
    TD = {0: torch.float64, 1: torch.float32, 2: torch.float16, 3: torch.bfloat16}
    g = torch.Generator(device="cuda")
    g.manual_seed(7)
    bits = torch.randint(-2 ** 31, 2 ** 31 - 1, (SRC_BYTES // 4,), dtype=torch.int32, device="cuda", generator=g)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for st, dt, name in DIRECTIONS:
        src = bits.view(TD[st])
        dst = torch.empty(src.numel(), dtype=TD[dt], device="cuda")
        for _ in range(2):
            flush.zero_()
            B.ps_convert(src, st, dst, dt)
        torch.cuda.synchronize()
        del dst


def summarise(path, out):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    ki, mi, vi, ui, idi = (hdr.index(k) for k in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit", "ID"))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "nsecond": 1e-9, "us": 1e-6,
             "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3}
    per = {}
    for r in rows[1:]:
        d = per.setdefault(int(r[idi]), {"name": r[ki]})
        d[r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
    launches = [per[k] for k in sorted(per) if "convert" in per[k]["name"]]
    res = {"source": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum "
                     "--clock-control none, tools/traffic_probe.py: 1 GiB of random bit patterns per "
                     "direction, L2 flushed, second launch of each", "directions": {}}
    for k, (st, dt, name) in enumerate(KERNEL_DIRECTIONS):
        d = launches[2 * k + 1]
        n = SRC_BYTES // SZ[st]
        alg = n * (SZ[st] + SZ[dt])
        dram = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
        res["directions"][name] = {
            "kernel": d["name"].split("(")[0], "algorithmic_bytes": alg, "dram_read": d.get("dram__bytes_read.sum"),
            "dram_write": d.get("dram__bytes_write.sum"), "ratio": round(dram / alg, 4),
            "us": round(d.get("gpu__time_duration.sum", 0) * 1e6, 2),
            "dram_GBps": round(dram / d["gpu__time_duration.sum"] / 1e9, 1) if d.get("gpu__time_duration.sum") else None}
    # the f32 -> f32 "conversion" of an inout object is a D2D copy (copy engine / driver
    # kernel, not ours): take the measured-copy ratio 1.0
    res["directions"]["f32->f32 copy"] = {"kernel": "cudaMemcpyAsync (D2D)", "ratio": 1.0,
                                         "note": "not a library kernel; algorithmic = DRAM bytes assumed"}
    json.dump(res, open(out, "w"), indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--summarise":
        summarise(sys.argv[2], sys.argv[3])
    else:
        run()
