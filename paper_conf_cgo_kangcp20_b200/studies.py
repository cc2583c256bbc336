"""Application-adaptivity studies on the CUDA path.

* ``fig6``  -- paper Fig. 6: the output quality of every app when ALL
  memory objects are fp16 (configuration id 3^M - 1), per input set (default,
  image, random), against TOQ 0.9.
* ``fig12`` -- paper Fig. 12: the Decision Maker's (Alg. 1 + PFP +
  wildcard, ``decision.decide``) whole-program speedup over the original fp32
  program (transfers included, ``ps_run_config_host``) and the fraction of
  objects it scales to fp16, per input set at TOQ 0.90 and for the default set
  at TOQ 0.90 / 0.95 / 0.99.  Beside it, the exhaustive device-only sweep's
  best passing configuration (``ps_sweep``) and its speedup over all-fp32.

Every number comes from the library (``binding``); this module only drives it.
``python -m paper_conf_cgo_kangcp20_b200.studies --out profiles/studies_r1.json``
"""
from __future__ import annotations

import argparse
import json
import sys
import time

from . import binding as B
from . import inputs as gen

# BASELINE sizes for the HBM-bound apps (N=16384); contractions at 2048 so that every
# app's full sweep + decision (with host transfers) finishes in seconds
SIZES = {"gemm": [2048], "2mm": [2048], "3mm": [1024], "atax": [16384, 16384], "bicg": [16384, 16384],
         "gesummv": [16384], "corr": [2048, 2048], "covar": [2048, 2048], "mvt": [16384],
         "syrk": [2048, 2048], "conv2d": [16384, 16384], "syr2k": [2048, 2048],
         "conv3d": [384, 384, 384], "fdtd2d": [20, 4096, 4096]}
INPUT_SETS = ("default", "image", "random")
TOQS = (0.90, 0.95, 0.99)


def _app(torch, kind, dims, iset):
    app = B.App(kind, dims)
    ins = gen.make_inputs(kind, app.objects, iset)
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    return app, ins


def fig6(torch, sizes=SIZES, input_sets=INPUT_SETS, toq=0.9):
    out = {}
    for kind, dims in sizes.items():
        row = {}
        for iset in input_sets:
            app, _ = _app(torch, kind, dims, iset)
            r = app.run_config([B.F16] * app.num_objects, toq)
            row[iset] = {"quality": round(r["quality"], 6), "pass": bool(r["pass"]),
                         "nonfinite": int(r["nonfinite"]), "max_rel": r["max_rel"]}
            del app
        out[kind] = row
    return out


def _device_best(app, toq):
    app.sweep_raw(list(range(app.space)), toq)      # warm-up: first launches load modules
    arr, bi = app.sweep_raw(list(range(app.space)), toq)
    f32 = arr[arr["config_id"] == app.encode([B.F32] * app.num_objects)]
    if bi < 0 or not len(f32):
        return None
    return {"best_prec": app.decode(int(arr["config_id"][bi])),
            "speedup_vs_f32": round(float(f32["total_ms"][0] / arr["total_ms"][bi]), 3),
            "passing": int(arr["pass"].sum()), "space": int(app.space)}


def fig12(torch, db, sizes=SIZES, cases=None, reps=5):
    from . import decision as D
    import numpy as np
    cases = cases or ([(iset, 0.90) for iset in INPUT_SETS] + [("default", 0.95), ("default", 0.99)])
    out = {}
    for kind, dims in sizes.items():
        row = {}
        for iset, toq in cases:
            app, ins = _app(torch, kind, dims, iset)
            host = [torch.from_numpy(x.reshape(-1)).pin_memory() if x is not None else None for x in ins]
            m = app.num_objects
            res = D.decide(app, host, db, toq=toq, reps=reps)
            orig = [app.run_config_host([B.F32] * m, host, [B.XFER_DEVICE] * m, toq=toq)["total_ms"]
                    for _ in range(reps)]
            mine = [app.run_config_host(res["prec"], host, res["methods"], toq=toq)["total_ms"]
                    for _ in range(reps)]
            row["%s@%.2f" % (iset, toq)] = {
                "chosen": res["prec"], "methods": res["method_names"],
                "half_fraction": round(sum(1 for p in res["prec"] if p == B.F16) / m, 4),
                "quality": round(res["result"]["quality"], 6),
                "original_f32_ms": round(float(np.median(orig)), 4),
                "chosen_ms": round(float(np.median(mine)), 4),
                "speedup": round(float(np.median(orig) / np.median(mine)), 3),
                "trials": res["trials"], "space": res["space"],
                "device_only_exhaustive": _device_best(app, toq)}
            del host, app
        out[kind] = row
    return out


def bf16_gain(torch, sizes=SIZES, input_sets=("default", "random"), toq=0.9):
    """the exhaustive device-only sweep over the paper's 3^M
    alphabet vs the bf16-extended 4^M one -- best passing speedup over all-fp32
    and the number of passing configurations.  bf16 keeps f32's exponent range,
    so objects that overflow fp16 (Fig. 6) can still take a 16-bit format and the
    tensor-core path."""
    out = {}
    for kind, dims in sizes.items():
        row = {}
        for iset in input_sets:
            app, _ = _app(torch, kind, dims, iset)
            base = _device_best(app, toq)
            app.set_flags(B.FLAG_BF16)
            ext = _device_best(app, toq)
            row[iset] = {"paper_3^M": base, "bf16_4^M": ext}
            del app
        out[kind] = row
    return out


def summarize(f12):
    """Geometric-mean speedup and mean fp16 fraction per case (Fig. 12 a-d)."""
    import math
    cases = sorted({c for row in f12.values() for c in row})
    out = {}
    for c in cases:
        sp = [row[c]["speedup"] for row in f12.values() if c in row]
        hf = [row[c]["half_fraction"] for row in f12.values() if c in row]
        out[c] = {"geomean_speedup": round(math.exp(sum(math.log(x) for x in sp) / len(sp)), 3),
                  "mean_half_fraction": round(sum(hf) / len(hf), 4), "apps": len(sp)}
    return out


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--apps", default=",".join(SIZES))
    ap.add_argument("--no-fig12", action="store_true")
    ap.add_argument("--bf16", action="store_true", help="also the radix-4 (bf16) sweep comparison")
    args = ap.parse_args(argv)
    import torch
    from . import decision as D
    torch.cuda.set_device(0)
    B.lib()
    sizes = {k: SIZES[k] for k in args.apps.split(",")}
    t0 = time.time()
    res = {"fig6_all_half_quality": fig6(torch, sizes)}
    print("fig6 done %.1f s" % (time.time() - t0), file=sys.stderr, flush=True)
    if not args.no_fig12:
        db = D.inspect(sizes=(1 << 20, 1 << 22, 1 << 24, 1 << 26), reps=2)
        res["fig12"] = fig12(torch, db, sizes)
        res["fig12_summary"] = summarize(res["fig12"])
        res["inspector_best_methods_2^26"] = {
            {0: "f64", 1: "f32", 2: "f16"}[dt]: D.NAMES[D.best_method(db, 1 << 26, dt)[0]] for dt in (0, 1, 2)}
    if args.bf16:
        res["bf16_gain"] = bf16_gain(torch, sizes)
    res["sizes"] = sizes
    res["seconds"] = round(time.time() - t0, 1)
    txt = json.dumps(res, indent=1)
    if args.out:
        with open(args.out, "w") as f:
            f.write(txt)
    print(txt)
    return 0


if __name__ == "__main__":
    sys.exit(main())
