#!/usr/bin/env python
"""Regenerate tests/golden/r5_rowdot.npz and tests/golden/r5_colsum.npz.

Calls ONLY oracle/ (and the seeded input generator): the goldens freeze the R5
reduction orders of DESIGN.md reading #21 so that no later change can silently
re-associate them ("R5 is frozen; any later change needs a new
reading and regenerated goldens, never a kernel convenience").

Workload: ATAX-shaped, A of NX = 2*256 + 37 rows (two full 256-row column-sum
chunks + a ragged chunk) by NY = 16384 + 37 columns (>= 16 row-dot tiles of
8 slabs at every A precision + a ragged slab), Random input set (P:160,
non-integer values in [0,1)), seed 2.  Configurations [A, x, y, tmp]:
  T = f32: A in {f64->no, f32, f16}, x/y/tmp f32 -> tmp = row-dot, y = column-sum, both in f32
  T = f64: A in {f64, f32, f16}, x/y/tmp f64     -> both in f64
(A in f64 with an f32 tmp would make T = f64, so the f32 set uses A f32/f16.)
Stored: the full row-dots (tmp, NX values), the column sums y at every 7th
column, and the SHA-256 of the full y bytes.
"""
import hashlib
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_cgo_kangcp20_b200 import inputs as gen  # noqa: E402

NX, NY = 2 * 256 + 37, 16384 + 37
SEED = 2
CONFIGS = {"f32_Af32": [1, 1, 1, 1], "f32_Af16": [2, 1, 1, 1],
           "f64_Af64": [0, 0, 0, 0], "f64_Af32": [1, 0, 0, 0], "f64_Af16": [2, 0, 0, 0]}


def compute():
    dims = [NX, NY]
    objs = oracle.app_objects("atax", dims)
    ins = gen.make_inputs("atax", objs, "random", seed=SEED)
    rowdot, colsum = {}, {}
    for name, prec in CONFIGS.items():
        fin = oracle.run_config("atax", dims, prec, ins)
        tmp = np.ascontiguousarray(fin[3].reshape(-1))
        y = np.ascontiguousarray(fin[2].reshape(-1))
        rowdot[name] = tmp
        colsum[name] = y[::7].copy()
        colsum[name + "_sha256"] = np.frombuffer(hashlib.sha256(y.tobytes()).digest(), dtype=np.uint8)
    return rowdot, colsum


def main():
    rowdot, colsum = compute()
    out = os.path.join(ROOT, "tests", "golden")
    np.savez(os.path.join(out, "r5_rowdot.npz"), nx=NX, ny=NY, seed=SEED, **rowdot)
    np.savez(os.path.join(out, "r5_colsum.npz"), nx=NX, ny=NY, seed=SEED, **colsum)
    print("wrote", out)


if __name__ == "__main__":
    main()
