#!/usr/bin/env python
"""bench.py -- PreScaler configuration-evaluation throughput on B200.

A "step" is one pass of the whole hot path over the
workload: for every app, the fp64 reference run (a0) and the evaluation of its
full configuration space 3^M (a1 decode, a2 conversion, a3 precision-scaled
kernels, a4+a5 fused back-conversion + quality, a6 records, a7 best config).
Default workload = BASELINE.json configs[2]: ATAX, BICG, GESUMMV at N=16384
(81 + 243 + 243 = 567 configurations per step), Table 4 "Default" inputs,
TOQ 0.9.  configs[1] (the conversion sweep) is a single row (a2) of the path,
so it is reported as the secondary `conversion_gbs` key, not as the step.

Multi-GPU (one process per GPU): ``--gpus N`` without a torchrun environment
re-executes this script under ``torch.distributed.run`` with N ranks (127.0.0.1
rendezvous); under torchrun (the driver's launch) the ranks come from the env.
The config space of every app is partitioned across ranks (deterministic LPT
over a cost model); each rank evaluates its share; one NCCL all_gather of the
64-byte result records per app per step; the contraction apps' fp64 reference
is row-sharded and all-gathered.  Timing: setup and warm-up first, then barrier
+ synchronize on both sides of exactly --steps steps, CUDA events on the
launching stream, max over ranks.  ``--backend gloo --fake`` is a CPU dry run of
the same orchestration (fake result records, no GPU) used by the CPU tests.

--impl reference times the CPU oracle (oracle/, the plain C definition) as it
stands on the host cores, on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    # BASELINE.json configs[2] (default)
    "matvec": [("atax", [16384, 16384]), ("bicg", [16384, 16384]), ("gesummv", [16384])],
    # BASELINE.json configs[0]
    "gemm64": [("gemm", [64])],
    # BASELINE.json configs[3] / configs[4] (3MM's 2187-config space at N=8192 is a
    # separate workload: one step is minutes of fp64 MMA on one GPU)
    "contract": [("2mm", [8192])],
    "contract3mm": [("3mm", [8192])],
    "corr": [("corr", [8192, 8192]), ("covar", [8192, 8192])],
    # SURVEY §8(f) NEXT #3 shapes at the mat-vec / contraction sizes of BASELINE
    "mvt": [("mvt", [16384])],
    "stencil": [("conv2d", [16384, 16384])],
    "syrk": [("syrk", [8192, 8192])],
    "syr2k": [("syr2k", [8192, 8192])],
    "stencil3d": [("conv3d", [512, 512, 512])],
    "fdtd": [("fdtd2d", [50, 8192, 8192])],
}
SIZE = {0: 8, 1: 4, 2: 2}
# CPU-oracle samples: (reduced dimension, work exponent) -- the oracle needs ~40 s
# per ATAX configuration at N=16384, so the CPU legs run every app dimension at
# the reduced size and extrapolate throughput by (N_sample / N)^exponent (O(N^2)
# mat-vec, O(N^3) contractions); labelled "extrapolated" in the JSON.
CPU_SAMPLE = {"matvec": (8192, 2), "gemm64": (None, 0), "contract": (384, 3), "contract3mm": (256, 3),
              "corr": (512, 3), "mvt": (8192, 2), "stencil": (4096, 2), "syrk": (512, 3),
              "syr2k": (384, 3), "stencil3d": (128, 3), "fdtd": (None, 0)}
# per-dimension sample overrides (the exponent then counts the scaled dimensions)
CPU_SAMPLE_DIMS = {"fdtd": [50, 1024, 1024]}
# GPU counts BASELINE.json names per workload (configs[2]: 1 and 2; [3]: 4; [4]: 8)
BASELINE_GPUS = {"matvec": [1, 2], "contract": [4], "contract3mm": [4], "corr": [8], "gemm64": [1]}
# BASELINE.md "paper context line": the paper's headline, other hardware -- context only
PAPER_CONTEXT = {
    "speedup": 1.33, "metric": "average whole-program speedup over the original precision at TOQ 0.9",
    "hardware": "Titan Xp + Xeon E5-2640v4, PCIe 3.0 x16, OpenCL 1.2", "workload": "14 PolyBench apps",
    "cite": "PAPER.md:388 (also 1.38x V100, 1.47x RTX 2080 Ti)", "context_only": True}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), float(p["bf16_tflops"]), "measured"
    except Exception:
        return 6650.0, 1590.0, "fallback"


# ------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index, self.proc = index, None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.FIELDS,
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            out, _ = self.proc.communicate(timeout=5)
        except Exception:
            self.proc.kill()
            out, _ = self.proc.communicate()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": float(max(mx)) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------- algorithmic bytes
def kernel_bytes(kind, dims, prec):
    """Algorithmic bytes of the a3 statement kernels of one configuration (one
    streaming pass over each matrix) + the vectors."""
    n = dims[0]
    if kind == "atax":
        return n * n * SIZE[prec[0]] + n * (SIZE[prec[1]] + SIZE[prec[2]] + 2 * SIZE[prec[3]])
    if kind == "bicg":
        return n * n * SIZE[prec[0]] + n * sum(SIZE[prec[k]] for k in (1, 2, 3, 4))
    if kind == "gesummv":
        return n * n * (SIZE[prec[0]] + SIZE[prec[1]]) + n * (SIZE[prec[2]] + 3 * SIZE[prec[3]] +
                                                            2 * SIZE[prec[4]])
    if kind == "mvt":      # one pass over A; x1, x2 read and written, y1, y2 read
        return n * n * SIZE[prec[0]] + n * (2 * SIZE[prec[1]] + 2 * SIZE[prec[2]] + SIZE[prec[3]] +
                                            SIZE[prec[4]])
    if kind == "conv2d":   # A read once, B written once
        return dims[0] * dims[1] * (SIZE[prec[0]] + SIZE[prec[1]])
    if kind == "conv3d":
        return dims[0] * dims[1] * dims[2] * (SIZE[prec[0]] + SIZE[prec[1]])
    if kind == "fdtd2d":   # per step: ey rd+wr, hz rd | ex rd+wr, hz rd | ex, ey rd, hz rd+wr
        return dims[0] * (dims[1] * dims[2] * (3 * SIZE[prec[1]] + 3 * SIZE[prec[2]] + 4 * SIZE[prec[3]]) +
                          dims[2] * SIZE[prec[2]])
    return None


# contraction statements: (a, b, out, M, N, K-flop-factor); SYRK computes the
# upper triangle only, so its algorithmic work is M*M*N multiply-adds / 2 * 2.
A3_KERNELS = {"atax": "tile_kernel + finalizers", "bicg": "tile_kernel + finalizers",
              "gesummv": "tile_kernel + finalizers + axpby", "mvt": "mvt tile_kernel + finalizers",
              "conv2d": "conv2d_kernel", "conv3d": "conv3d_kernel",
              "fdtd2d": "fdtd_ey/ex/hz_kernel x TMAX"}


def _contractions(kind, d):
    if kind == "gemm":
        return [(0, 1, 2, d[0], d[1], d[2])]
    if kind == "2mm":
        return [(0, 1, 2, d[0], d[1], d[2]), (2, 3, 4, d[0], d[3], d[1])]
    if kind == "3mm":
        return [(0, 1, 4, d[0], d[1], d[2]), (2, 3, 5, d[1], d[3], d[4]), (4, 5, 6, d[0], d[3], d[1])]
    if kind in ("corr", "covar"):
        return [(0, 0, 3 if kind == "corr" else 2, d[1], d[1], d[0] / 2.0)]
    if kind == "syrk":
        return [(0, 0, 1, d[1], d[1], d[0] / 2.0)]
    if kind == "syr2k":
        return [(0, 1, 2, d[1], d[1], d[0]), (1, 0, 2, d[1], d[1], d[0])]
    return []


def contraction_roofline(apps, last):
    """a3 of contraction workloads: frac = sum of ideal statement times (flops / the
    peak of the pipe the statement runs on) / sum of measured kernel times.  Peaks:
    tensor = MEASURED_PEAKS bf16 burst (fp16 has the same dense rate); FFMA and f64
    derived from unit counts (128 / 64 FMA per SM per clock) x 148 SMs x 1965 MHz
    (f64 statements run on the fp64 tensor-core MMA, DMMA: measured 37.0 TFLOP/s on a
    pure-MMA loop, profiles/dmma_probe_r1.txt, so the derived 37.2 is the ceiling)."""
    _, tc_peak, _ = measured_peaks()
    peaks = {"tensor": tc_peak, 1: 148 * 128 * 2 * 1.965e9 / 1e12, 0: 148 * 64 * 2 * 1.965e9 / 1e12}
    ideal = meas = flops = 0.0
    paths = {}
    for a in apps:
        dims = a["dims"] if len(a["dims"]) > 1 else a["dims"] * 5
        sts = _contractions(a["kind"], dims)
        if not sts:
            return None
        m = a["app"].num_objects
        for r in last[a["kind"]]:
            p = decode(int(r["config_id"]), m)
            for (x, y, o, M, N, K) in sts:
                T = 0 if 0 in (p[x], p[y], p[o]) else 1
                path = "tensor" if (p[x] == 2 and p[y] == 2 and T == 1) else T
                f = 2.0 * M * N * K
                flops += f
                ideal += f / (peaks[path] * 1e12)
                paths[str(path)] = paths.get(str(path), 0) + 1
            meas += float(r["kernel_ms"]) * 1e-3
    if meas <= 0:
        return None
    return {"bound": "tensor+fma", "achieved": round(flops / meas / 1e12, 2), "unit": "TFLOP/s",
            "peak": {"tensor": tc_peak, "ffma": round(peaks[1], 1), "f64_dmma": round(peaks[0], 1)},
            "frac": round(ideal / meas, 4), "traffic": None,
            "peak_source": "tensor: MEASURED_PEAKS.json bf16_tflops (burst); FMA pipes derived",
            "kernel": "a3 contraction statements (gemm_tc2_kernel fp16/bf16/fp8, gemm_dmma_kernel f64, gemm_simt_kernel f32)",
            "statements_by_path": paths}


# FP ops per output of the ALU-heavy stencils (products rounded separately, R4):
# 3DCONV 27 multiplies + 26 adds (reading #26)
STENCIL_OPS = {"conv3d": 53}


def stencil_roofline(apps, last, hbm):
    """a3 of 3DCONV: per configuration the ideal time is max(ALU time, HBM time) with
    ALU peak = FP32 (128) or FP64 (64) lanes/clk/SM x 148 SMs x 1965 MHz (one lane-op
    per FMUL/FADD) and HBM = the measured copy bandwidth; frac = sum ideal / sum measured."""
    lanes = {1: 148 * 128 * 1.965e9, 0: 148 * 64 * 1.965e9}
    ideal = meas = ops = 0.0
    bound_t = {"alu": 0.0, "hbm": 0.0}
    for a in apps:
        k = a["kind"]
        if k not in STENCIL_OPS:
            return None
        m = a["app"].num_objects
        n_out = float(np.prod(a["dims"]))
        for r in last[k]:
            p = decode(int(r["config_id"]), m)
            T = 0 if 0 in p else 1
            t_alu = n_out * STENCIL_OPS[k] / lanes[T]
            t_hbm = kernel_bytes(k, a["dims"], p) / (hbm * 1e9)
            ideal += max(t_alu, t_hbm)
            bound_t["alu" if t_alu >= t_hbm else "hbm"] += max(t_alu, t_hbm)
            ops += n_out * STENCIL_OPS[k]
            meas += float(r["kernel_ms"]) * 1e-3
    if meas <= 0:
        return None
    return {"bound": max(bound_t, key=bound_t.get), "achieved": round(ops / meas / 1e12, 3),
            "unit": "TFLOP/s (FP32/FP64 lane-ops)", "peak": {"fp32": round(lanes[1] / 1e12, 1),
                                                              "fp64": round(lanes[0] / 1e12, 1),
                                                              "hbm_gbs": hbm},
            "frac": round(ideal / meas, 4), "traffic": None,
            "peak_source": "ALU peaks derived from unit counts (B200_PROFILING.md: 148 SMs, 1965 MHz); "
                           "HBM = MEASURED_PEAKS.json; ideal per config = max(ALU, HBM) time",
            "kernel": "a3 conv3d_kernel (2.5-D smem blocking, cp.async ring)",
            "ideal_time_share": {k2: round(v / ideal, 4) for k2, v in bound_t.items()}}


CNAME = {0: "f32->f64", 1: "f32->f32 copy", 2: "f32->f16", 3: "f32->bf16"}


def convert_bytes(objects, prec, by_dir=None):
    """Algorithmic bytes of one configuration's a2 conversions (orig f32 -> c(m) for every
    object read before written; inout objects are copied even at f32); by_dir (dict)
    receives the bytes per direction."""
    b = 0
    for o, p in zip(objects, prec):
        if o["role"] in (0, 2) and (p != 1 or o["role"] == 2):
            x = o["n"] * (4 + SIZE[p])
            b += x
            if by_dir is not None:
                by_dir[CNAME[p]] = by_dir.get(CNAME[p], 0) + x
    return b


def decode(cid, m):
    out = []
    for _ in range(m):
        out.append(cid % 3)
        cid //= 3
    return out


# ---------------------------------------------------------- reference arm
def _sample(workload):
    kind, dims = WORKLOADS[workload][0]
    n_s, expo = CPU_SAMPLE[workload]
    if workload in CPU_SAMPLE_DIMS:
        sdims = CPU_SAMPLE_DIMS[workload]
        factor = float(np.prod(sdims)) / float(np.prod(dims))
        return kind, dims, sdims, factor, 1
    sdims = dims if n_s is None else [n_s] * len(dims)
    factor = 1.0 if n_s is None else (n_s / float(dims[0])) ** expo
    return kind, dims, sdims, factor, expo


def _oracle_batch(kind, sdims, ins, ref, ids, toq, threads):
    """Evaluate configurations with the oracle, one per host thread (ctypes releases
    the GIL inside the C oracle, which keeps no global state)."""
    import oracle
    from concurrent.futures import ThreadPoolExecutor
    m = len(oracle.app_objects(kind, sdims))
    if threads <= 1:
        for c in ids:
            oracle.evaluate(kind, sdims, decode(c, m), ins, ref, toq=toq)
        return
    with ThreadPoolExecutor(threads) as ex:
        list(ex.map(lambda c: oracle.evaluate(kind, sdims, decode(c, m), ins, ref, toq=toq), ids))


def _cycle_ids(m, k, start):
    space = 3 ** m
    return [(start + 7 * i) % space for i in range(k)]


def run_reference_arm(args, rank, world):
    """The CPU oracle as it stands, one configuration per host core in parallel,
    on a bounded sample per step."""
    import oracle
    from paper_conf_cgo_kangcp20_b200 import inputs as gen
    if rank != 0:
        return 0
    kind, dims, sdims, factor, expo = _sample(args.workload)
    objs = oracle.app_objects(kind, sdims)
    ins = gen.make_inputs(kind, objs, args.input_set)
    cores = os.cpu_count() or 1
    t0 = time.time()
    ref = oracle.reference(kind, sdims, ins)
    t_ref = time.time() - t0
    m = len(objs)
    for w in range(args.warmup):
        _oracle_batch(kind, sdims, ins, ref, _cycle_ids(m, cores, w * cores), args.toq, cores)
    t0 = time.time()
    for s in range(args.steps):
        _oracle_batch(kind, sdims, ins, ref, _cycle_ids(m, cores, (args.warmup + s) * cores), args.toq,
                      cores)
    el = time.time() - t0
    v = args.steps * cores / el * factor
    sample = "%s %s: per step %d configurations (ids 7i+c mod 3^M), one per host thread, at %s, " \
             "fp64 reference precomputed (%.1f s); throughput extrapolated to %s by (N_s/N)^%d = %.4g" % (
                 kind, "x".join(map(str, dims)), cores, "x".join(map(str, sdims)), t_ref,
                 "x".join(map(str, dims)), expo, factor)
    line = {"impl": "reference", "metric": "configs evaluated/s", "value": v,
            "unit": "configs/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": el / args.steps * 1e3, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64/f32/f16 (per configuration)", "data": "synthetic",
            "config": {"workload": args.workload, "sample": sample, "input_set": args.input_set,
                       "toq": args.toq},
            "cpu_baseline": {"value": v, "unit": "configs/s", "cores": cores, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": v, "unit": "configs/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def cpu_baseline(args):
    """Oracle timed on the host: the fp64 reference run, then one
    configuration single-threaded and a batch of one configuration per host core in
    parallel, at the sample size; value = the parallel rate."""
    import oracle
    from paper_conf_cgo_kangcp20_b200 import inputs as gen
    kind, dims, sdims, factor, expo = _sample(args.workload)
    objs = oracle.app_objects(kind, sdims)
    ins = gen.make_inputs(kind, objs, args.input_set)
    m = len(objs)
    cores = os.cpu_count() or 1
    t0 = time.time()
    ref = oracle.reference(kind, sdims, ins)
    t_ref = time.time() - t0
    t0 = time.time()
    _oracle_batch(kind, sdims, ins, ref, [(3 ** m - 1) // 2], args.toq, 1)
    t_one = time.time() - t0
    ids = _cycle_ids(m, cores, 1)
    t0 = time.time()
    _oracle_batch(kind, sdims, ins, ref, ids, args.toq, cores)
    t_par = time.time() - t0
    lscpu = ""
    try:
        lscpu = [l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name")][0]
    except Exception:
        pass
    return {"value": cores / t_par * factor, "unit": "configs/s", "cores": cores, "kind": "oracle",
            "cpu_model": lscpu,
            "single_thread": {"value": 1.0 / t_one * factor, "cores": 1},
            "sample": "%s at %s: fp64 reference %.1f s; all-f32 config single-threaded %.1f s; %d configs "
                      "(ids 7i+1 mod 3^M) one per thread in %.1f s; plain C oracle; extrapolated to %s by "
                      "(N_s/N)^%d = %.4g" % (kind, "x".join(map(str, sdims)), t_ref, t_one, cores, t_par,
                                             "x".join(map(str, dims)), expo, factor)}


# ------------------------------------------------------- whole program
def whole_program(torch, B, apps, args):
    """The paper's end metric: the Decision Maker's configuration (precisions +
    conversion methods chosen from a System Inspector DB measured here) vs the original
    program (every object f32, transferred as f32), both run from pinned host inputs
    with ps_run_config_host (transfers included).  Not part of the timed value."""
    from paper_conf_cgo_kangcp20_b200 import decision as D
    t0 = time.time()
    db = D.inspect(sizes=(1 << 20, 1 << 24, 1 << 26), reps=2)
    out = {"inspector_s": None, "apps": {}}
    out["inspector_s"] = round(time.time() - t0, 2)
    out["best_methods_n2^26"] = {
        {0: "f64", 1: "f32", 2: "f16"}[dt]: D.NAMES[D.best_method(db, 1 << 26, dt)[0]] for dt in (0, 1, 2)}
    for a in apps:
        app = a["app"]
        host = [torch.from_numpy(x.reshape(-1)).pin_memory() if x is not None else None for x in a["ins"]]
        m = app.num_objects
        res = D.decide(app, host, db, toq=args.toq, reps=3)
        orig = [app.run_config_host([1] * m, host, [0] * m, toq=args.toq)["total_ms"] for _ in range(3)]
        mine = [app.run_config_host(res["prec"], host, res["methods"], toq=args.toq)["total_ms"]
                for _ in range(3)]
        out["apps"][a["kind"]] = {
            "original_f32_ms": round(float(np.median(orig)), 3),
            "chosen": {"prec": res["prec"], "methods": res["method_names"]},
            "chosen_ms": round(float(np.median(mine)), 3),
            "speedup": round(float(np.median(orig) / np.median(mine)), 3),
            "trials": res["trials"], "space": res["space"],
            "quality": round(res["result"]["quality"], 6)}
        del host
    return out


# ------------------------------------------------------------ conversion
CONV_DIRECTIONS = [(1, 2, "f32->f16"), (2, 1, "f16->f32"), (0, 2, "f64->f16"), (0, 1, "f64->f32"),
                   (1, 0, "f32->f64"), (1, 3, "f32->bf16")]
CSIZE = {0: 8, 1: 4, 2: 2, 3: 2}


def random_bits(torch, nbytes):
    """Uniform random bit patterns (every class: normals, subnormals, +-inf, NaNs), so the
    measured speed is value-independent."""
    g = torch.Generator(device="cuda")
    g.manual_seed(20200222)
    n = nbytes // 4
    return torch.randint(-2 ** 31, 2 ** 31 - 1, (n,), dtype=torch.int32, device="cuda", generator=g)


def conversion_sweep(torch, B, flush, reps=20, sizes=None):
    """BASELINE configs[1] / SURVEY §8(d)-2 row 2: source sizes 2^20 .. 2^32 bytes, the four
    BASELINE directions plus f32->f64 (the a2 direction of every f64 configuration) and
    f32->bf16, random bit patterns, L2 flushed before every rep, median of `reps` CUDA-event
    timings.  Algorithmic GB/s = n (s_src + s_dst) / t."""
    sizes = sizes or [1 << k for k in range(20, 33)]
    out = {}
    TD = {0: torch.float64, 1: torch.float32, 2: torch.float16, 3: torch.bfloat16}
    bits = random_bits(torch, max(sizes))
    for st, dt, name in CONV_DIRECTIONS:
        row = {}
        for nbytes in sizes:
            n = nbytes // CSIZE[st]
            src = bits[:nbytes // 4].view(TD[st])[:n]
            dst = torch.empty(n, dtype=TD[dt], device="cuda")
            for _ in range(3):
                B.ps_convert(src, st, dst, dt)
            ts = []
            for _ in range(reps):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                B.ps_convert(src, st, dst, dt)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            t = float(np.median(ts))
            row[nbytes] = round(n * (CSIZE[st] + CSIZE[dt]) / (t * 1e-3) / 1e9, 1)
            del dst
        out[name] = row
    del bits
    return out


# ------------------------------------------------------------- launching
def _free_port() -> int:
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def spawn_ranks(n: int) -> int:
    """`bench.py --gpus N` outside torchrun: re-run this script as N ranks (one
    process per GPU) under torch.distributed.run; rank 0 prints the line."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(n),
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
           os.path.abspath(__file__)] + sys.argv[1:]
    log("spawning %d ranks: %s" % (n, " ".join(cmd)))
    return subprocess.call(cmd)


def fake_records(ids, costs):
    """--fake: deterministic stand-in for ps_sweep records (CPU dry run, no GPU):
    total_ms = the cost model's prediction, quality from the id."""
    import paper_conf_cgo_kangcp20_b200.binding as B
    rec = np.zeros(len(ids), dtype=B.RESULT_DTYPE)
    rec["config_id"] = np.asarray(ids, dtype=np.uint64)
    rec["total_ms"] = np.asarray(costs, dtype=np.float32) * 1e3
    rec["quality"] = 1.0 - (np.asarray(ids, dtype=np.uint64) * np.uint64(2654435761) % np.uint64(1000)) / 5e3
    rec["pass"] = (rec["quality"] >= 0.9).astype(np.int32)
    return rec


def run_fake(args, rank, world):
    """The multi-rank orchestration of the real run -- partition, per-rank sweep,
    record gather, best config, max-over-ranks timing, one line from rank 0 --
    with fake records and the gloo backend, so it runs (and is tested) on CPU."""
    import torch
    import torch.distributed as dist

    from paper_conf_cgo_kangcp20_b200 import binding as B
    from paper_conf_cgo_kangcp20_b200 import dist as D
    if world > 1:
        dist.init_process_group(args.backend)
    apps = []
    for kind, dims in WORKLOADS[args.workload]:
        app = B.App(kind, dims)          # host metadata only
        ids = list(range(app.space))
        mine = D.partition_configs(kind, dims, app.objects, ids, world, rank) if world > 1 else ids
        costs = [D.config_cost(kind, dims, app.objects, c) for c in mine]
        apps.append(dict(kind=kind, ids=mine, costs=costs, space=app.space))
    total = sum(a["space"] for a in apps)

    def step():
        best = {}
        for a in apps:
            arr = fake_records(a["ids"], a["costs"])
            if world > 1:
                arr = D.gather_results(arr)
            assert len(arr) == a["space"]
            best[a["kind"]] = int(arr["config_id"][D.best_index(arr)]) if D.best_index(arr) >= 0 else -1
        return best

    for _ in range(args.warmup):
        step()
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        best = step()
    el = time.perf_counter() - t0
    el_t = torch.tensor([el], dtype=torch.float64)
    counts = torch.tensor([sum(len(a["ids"]) for a in apps)], dtype=torch.int64)
    allc = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
    if world > 1:
        dist.all_reduce(el_t, op=dist.ReduceOp.MAX)
        dist.all_gather(allc, counts)
    else:
        allc = [counts]
    if rank == 0:
        line = {"metric": "configs evaluated/s", "value": total * args.steps / el_t.item(),
                "unit": "configs/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": el_t.item() / args.steps * 1e3, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "none (fake records)",
                "data": "FAKE: CPU dry run of the multi-rank orchestration, no GPU, not a measurement",
                "fake": True, "backend": args.backend,
                "config": {"workload": args.workload, "configs_per_step": total,
                           "configs_per_rank": [int(c.item()) for c in allc], "best_config": best}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


# ------------------------------------------------------------------- main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="matvec", choices=sorted(WORKLOADS))
    ap.add_argument("--input-set", default="default", choices=["default", "random", "image"])
    ap.add_argument("--toq", type=float, default=0.9)
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"])
    ap.add_argument("--fake", action="store_true",
                    help="CPU dry run of the multi-rank orchestration (fake records; needs --backend gloo)")
    ap.add_argument("--shard-rows", action="store_true",
                    help="evaluate every configuration row-sharded over all ranks (ps_shard_step) "
                         "instead of partitioning the configurations")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-conversion", action="store_true")
    ap.add_argument("--no-whole-program", action="store_true")
    ap.add_argument("--profile", action="store_true",
                    help="one untimed-warmup-free step for ncu launch lists (not a bench number)")
    args = ap.parse_args()
    if args.profile:
        args.warmup, args.steps = 0, 1
        args.no_e2e = args.no_cpu_baseline = args.no_conversion = True
    elif args.warmup < 3:
        log("warmup raised to 3 (timing rule)")
        args.warmup = 3
    if args.shard_rows:
        args.no_e2e = True
    if args.fake and args.backend != "gloo":
        ap.error("--fake runs on CPU: use --backend gloo")

    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "ours":
        return spawn_ranks(args.gpus)
    rank, world = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if world != args.gpus and args.impl == "ours":
        log("note: --gpus %d but WORLD_SIZE %d; the run uses %d rank(s)" % (args.gpus, world, world))
    if args.impl == "reference":
        return run_reference_arm(args, rank, world)
    if args.fake:
        return run_fake(args, rank, world)

    import torch
    import torch.distributed as dist

    from paper_conf_cgo_kangcp20_b200 import binding as B
    from paper_conf_cgo_kangcp20_b200 import build as build_mod
    from paper_conf_cgo_kangcp20_b200 import dist as D
    from paper_conf_cgo_kangcp20_b200 import inputs as gen

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group(args.backend, device_id=torch.device("cuda", local))
    if rank == 0:
        build_mod.build()
    if world > 1:
        dist.barrier()
    B.lib()
    stream = torch.cuda.current_stream()

    # ------------------------------------------------------------ setup (a0 inputs)
    apps = []
    for kind, dims in WORKLOADS[args.workload]:
        app = B.App(kind, dims)
        t0 = time.time()
        ins = gen.make_inputs(kind, app.objects, args.input_set)
        dins = [torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins]
        app.bind(dins)
        refs = D.sharded_reference(app, world, rank)
        ids = list(range(app.space))
        mine = D.partition_configs(kind, dims, app.objects, ids, world, rank) if world > 1 and not args.shard_rows else ids
        apps.append(dict(kind=kind, dims=dims, app=app, ins=ins, refs=refs, ids=mine,
                         space=app.space))
        log("rank %d setup %s %s: %d/%d configs, %.1f s" % (rank, kind, dims, len(mine),
                                                              app.space, time.time() - t0))
    total_configs = sum(a["space"] for a in apps)
    max_obj = max(o["n"] * 4 for a in apps for o in a["app"].objects)

    def step(collect=None):
        for a in apps:
            D.sharded_reference(a["app"], world, rank, refs=a["refs"])   # a0 (row-sharded)
            if args.shard_rows:
                # every configuration row-sharded over all ranks (ps_shard_step stages +
                # NCCL all-gathers of the exchanged ranges), records identical on every rank
                recs = [D.sharded_evaluate(a["app"], a["app"].decode(c), args.toq) for c in range(a["space"])]
                arr = np.zeros(len(recs), dtype=B.RESULT_DTYPE)
                for i, r in enumerate(recs):
                    for k in B.RESULT_DTYPE.names:
                        arr[i][k] = r[k]
            else:
                arr, _ = a["app"].sweep_raw(a["ids"], args.toq)      # a1-a7 (local share)
                if world > 1:
                    arr = D.gather_results(arr)                      # NCCL gather
            if collect is not None:
                collect[a["kind"]] = arr

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    # ----------------------------------------------------------------- timed
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    last = {}
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = B.ps_kernel_launches()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for s in range(args.steps):
        step(last if s == args.steps - 1 else None)
    e1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = B.ps_kernel_launches() - l0
    el_ms = e0.elapsed_time(e1)
    clk = clocks.stop()
    if world > 1:
        t = torch.tensor([el_ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        el_ms = float(t.item())
        lt = torch.tensor([launches], dtype=torch.int64, device="cuda")
        dist.all_reduce(lt, op=dist.ReduceOp.SUM)
        launches = int(lt.item())
    value = total_configs * args.steps / (el_ms * 1e-3)
    per_rank = [sum(len(a["ids"]) for a in apps)]
    if world > 1:
        c = torch.tensor([per_rank[0]], dtype=torch.int64, device="cuda")
        allc = torch.zeros(world, dtype=torch.int64, device="cuda")
        dist.all_gather_into_tensor(allc, c)
        per_rank = [int(x) for x in allc.cpu().tolist()]

    # ------------------------------------------------- e2e through host buffers
    e2e = None
    if not args.no_e2e:
        host = []
        h2d = 0
        for a in apps:
            hin = [torch.from_numpy(x.reshape(-1)).pin_memory() if x is not None else None
                   for x in a["ins"]]
            host.append(hin)
            h2d += sum(x.numel() * 4 for x in hin if x is not None)
        d2h = sum(len(a["ids"]) * 24 for a in apps)      # one (sum e, max, count) record per config

        copy = torch.cuda.Stream()
        # two device input sets per app: step k sweeps set k % 2 while step k+1's inputs
        # cross PCIe into the other set (every step still copies all of its inputs
        # inside the timed region; only the first copy of the run is exposed)
        sets = []
        for a in apps:
            cur = a["app"].inputs
            sets.append([cur, [torch.empty_like(t) if t is not None else None for t in cur]])

        def issue_copies(k):
            """H2D of step k's inputs into set k % 2 on the copy stream; one event per app."""
            go = torch.cuda.Event()
            go.record(stream)                        # the previous user of that set is done
            copy.wait_event(go)
            evs = []
            for i, (a, hin) in enumerate(zip(apps, host)):
                dst = sets[i][k % 2]
                a["app"].bind(dst, outputs=a["app"].outputs, workspace=a["app"].workspace)
                a["app"].load_host(hin, stream=copy)                 # H2D into set k % 2
                ev = torch.cuda.Event()
                ev.record(copy)
                evs.append(ev)
            return evs

        def step_e2e(k, ready, last):
            nxt = None if last else issue_copies(k + 1)
            for i, (a, ev) in enumerate(zip(apps, ready)):
                a["app"].bind(sets[i][k % 2], outputs=a["app"].outputs, workspace=a["app"].workspace)
                stream.wait_event(ev)
                D.sharded_reference(a["app"], world, rank, refs=a["refs"])
                arr, _ = a["app"].sweep_raw(a["ids"], args.toq)       # results read back (D2H)
                if world > 1:
                    D.gather_results(arr)
            return nxt

        ready = issue_copies(0)                      # warm-up step
        step_e2e(0, ready, True)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        ready = issue_copies(0)
        for k in range(args.steps):
            ready = step_e2e(k, ready, k == args.steps - 1)
        f1.record(stream)
        torch.cuda.synchronize()
        e_ms = f0.elapsed_time(f1)
        if world > 1:
            t = torch.tensor([e_ms], dtype=torch.float64, device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e_ms = float(t.item())
        e2e = {"value": total_configs * args.steps / (e_ms * 1e-3), "unit": "configs/s",
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": e_ms / args.steps,
               "how": "ps_app_load_host of every input (pinned f32) each step on a copy stream into one of "
                      "two device input sets, overlapped with the previous step's sweep; ps_sweep reads "
                      "the result records back each app"}
        del host

    if rank != 0:
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()
        return 0

    # -------------------------------------------------------- roofline & shares
    hbm, _, peak_src = measured_peaks()
    phase = {"convert": 0.0, "kernel": 0.0, "backconv": 0.0, "quality": 0.0}
    kb = kt = cb = ct = 0.0
    conv_dirs = {}
    speedup = {}
    n_kernel_groups = 0
    for a in apps:
        arr = last[a["kind"]]
        m = a["app"].num_objects
        phase["convert"] += float(arr["convert_ms"].sum())
        phase["kernel"] += float(arr["kernel_ms"].sum())
        phase["backconv"] += float(arr["backconv_ms"].sum())
        phase["quality"] += float(arr["quality_ms"].sum())
        for r in arr:
            prec = decode(int(r["config_id"]), m)
            b = kernel_bytes(a["kind"], a["dims"], prec)
            if b is not None:
                kb += b
                kt += float(r["kernel_ms"])
                n_kernel_groups += 1
            c = convert_bytes(a["app"].objects, prec, conv_dirs)
            if c:
                cb += c
                ct += float(r["convert_ms"])
        f32 = arr[arr["config_id"] == (3 ** m - 1) // 2]
        bi = D.best_index(arr)
        if len(f32) and bi >= 0:
            speedup[a["kind"]] = {
                "all_f32_ms": round(float(f32["total_ms"][0]), 4),
                "best_id": int(arr["config_id"][bi]), "best_prec": decode(int(arr["config_id"][bi]), m),
                "best_ms": round(float(arr["total_ms"][bi]), 4),
                "speedup": round(float(f32["total_ms"][0] / arr["total_ms"][bi]), 3),
                "passing": int(arr["pass"].sum()), "configs": int(len(arr))}
    ratios = {}
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        try:
            ratios = json.load(open(tp))
        except Exception:
            ratios = {}
    psrc = (peak_src + " (MEASURED_PEAKS.json hbm_gbs)") if peak_src == "measured" \
        else "fallback (B200_PROFILING.md)"

    # measured DRAM bytes / algorithmic bytes per conversion direction (ncu, 1 GiB launches,
    # tools/traffic_probe.py -> profiles/ncu_traffic_convert_r2.json), weighted by this
    # step's bytes per direction
    conv_ratio, conv_ratio_src = None, None
    tpc = os.path.join(ROOT, "profiles", "ncu_traffic_convert_r2.json")
    if os.path.exists(tpc) and conv_dirs:
        try:
            dirs = json.load(open(tpc))["directions"]
            if all(k in dirs for k in conv_dirs):
                conv_ratio = sum(dirs[k]["ratio"] * v for k, v in conv_dirs.items()) / sum(conv_dirs.values())
                conv_ratio_src = "profiles/ncu_traffic_convert_r2.json, weighted by %s" % (
                    {k: round(v / sum(conv_dirs.values()), 4) for k, v in conv_dirs.items()})
        except Exception:
            conv_ratio = None
    if conv_ratio is not None:
        ratios["convert_ratio"] = conv_ratio

    def hbm_roof(bytes_, ms_, n_, kernel, ratio_key):
        if ms_ <= 0 or n_ == 0:
            return None
        ach = bytes_ / (ms_ * 1e-3) / 1e9
        per = bytes_ / n_
        r = ratios.get(ratio_key)
        out = {"bound": "hbm", "achieved": round(ach, 1), "peak": hbm, "unit": "GB/s",
               "frac": round(ach / hbm, 4), "traffic": round(r * per) if r else None,
               "peak_source": psrc, "kernel": kernel,
               "algorithmic_bytes_per_launch": round(per), "avg_launch_ms": round(ms_ / n_, 5)}
        if ratio_key == "convert_ratio":
            out["traffic_source"] = conv_ratio_src or ratios.get("convert_source")
            out["bytes_by_direction"] = {k: int(v) for k, v in conv_dirs.items()}
        else:
            out["traffic_source"] = ratios.get("source")
        return out

    n_conv_groups = sum(1 for a in apps for r in last[a["kind"]]
                        if convert_bytes(a["app"].objects, decode(int(r["config_id"]), a["app"].num_objects)))
    knames = sorted({A3_KERNELS.get(a["kind"], a["kind"]) for a in apps})
    roof_a3 = hbm_roof(kb, kt, n_kernel_groups,
                       "a3 statement kernels of one configuration (%s)" % ", ".join(knames), "ratio")
    roof_a2 = hbm_roof(cb, ct, n_conv_groups,
                       "a2 conversion kernels of one configuration (convert_bulk_kernel: TMA bulk "
                       "load/store ring)", "convert_ratio")
    roof_mm = contraction_roofline(apps, last) if kb == 0 else None
    roof_st = stencil_roofline(apps, last, hbm)
    # the dominant phase's kernel is THE roofline; the other is reported beside it
    if roof_mm is not None:
        roof, conv_roof = roof_mm, roof_a2
    elif roof_st is not None:
        roof, conv_roof = roof_st, roof_a3
    elif phase["convert"] > phase["kernel"] and roof_a2 is not None:
        roof, conv_roof = roof_a2, roof_a3
    else:
        roof, conv_roof = roof_a3, roof_a2

    # modelled multi-GPU scaling (labelled as a model, not a measurement): the partition
    # dist.partition_configs would use at W ranks (LPT over the cost model), applied to
    # this run's MEASURED per-configuration device times; the makespan is the slowest
    # rank's sum.  Excludes the NCCL record gather (64 B per configuration) and setup.
    scaling_model = None
    if world == 1:
        scaling_model = {"how": "LPT partition of the cost model (dist.partition_configs) applied to this "
                                "run's measured per-configuration total_ms; makespan = slowest rank; "
                                "model, not a measurement", "speedup": {}}
        t1 = sum(float(last[a["kind"]]["total_ms"].sum()) for a in apps)
        for W in (2, 4, 8):
            ranks = [0.0] * W
            for a in apps:
                arr = last[a["kind"]]
                ms = {int(c): float(t) for c, t in zip(arr["config_id"], arr["total_ms"])}
                ids = sorted(ms)
                for r in range(W):
                    part = D.partition_configs(a["kind"], a["dims"], a["app"].objects, ids, W, r)
                    ranks[r] += sum(ms[c] for c in part)
            scaling_model["speedup"][str(W)] = round(t1 / max(ranks), 3)

    whole = None
    if not args.no_whole_program and world == 1:
        whole = whole_program(torch, B, apps, args)

    cpu = None
    if not args.no_cpu_baseline and world == 1:
        cpu = cpu_baseline(args)

    conv = None
    if not args.no_conversion:
        flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
        sweep = conversion_sweep(torch, B, flush)
        conv = {k: {"gbs": v[1 << 30], "frac_of_measured": round(v[1 << 30] / hbm, 4),
                    "frac_of_8tbs": round(v[1 << 30] / 8000, 4),
                    "min_frac_at_ge_256MB": round(min(g for b, g in v.items() if b >= 256 << 20) / hbm, 4),
                    "sweep_gbs_by_src_bytes": {str(b): g for b, g in v.items()}}
                for k, v in sweep.items()}

    tot_phase = sum(phase.values())
    line = {
        "metric": "configs evaluated/s", "value": round(value, 2), "unit": "configs/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(el_ms / args.steps, 4), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None,
        "dtype": "f64/f32/f16 (per memory object, per configuration)", "data": "synthetic",
        "config": {"workload": args.workload,
                   "apps": ["%s %s" % (a["kind"], "x".join(map(str, a["dims"]))) for a in apps],
                   "configs_per_step": total_configs, "input_set": args.input_set, "toq": args.toq,
                   "step": "a0 reference + full 3^M config space per app (a1-a7)",
                   "l2": "inputs larger than L2: largest object %.0f MB at fp32 vs 126 MB L2%s" % (
                       max_obj / 1e6, "" if max_obj > 126e6 else " (NOT larger: launch-bound case)"),
                   "parallelism": ("each configuration row-sharded over %d GPU(s) (ps_shard_step, NCCL "
                                   "all-gathers of the exchanged ranges)" % world) if args.shard_rows else
                                  "configs partitioned over %d GPU(s), NCCL result gather" % world,
                   "configs_per_rank": per_rank,
                   "baseline_n_gpus": BASELINE_GPUS.get(args.workload)},
        "paper_context": PAPER_CONTEXT,
        "e2e": e2e, "gpu_launches": launches,
        "roofline": roof, "cpu_baseline": cpu, "clocks": clk,
        "phase_share": {k: round(v / tot_phase, 4) for k, v in phase.items()} if tot_phase else None,
        "roofline_secondary": conv_roof,
        "conversion_gbs": conv,
        "speedup_vs_fp32_at_toq": speedup,
        "scaling_model": scaling_model,
        "whole_program": whole,
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
