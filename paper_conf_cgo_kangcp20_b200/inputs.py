"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module holds none of the method's arithmetic: it only produces the
original-precision (fp32, reading #13) contents of each input memory object.
The recipe:

* ``default`` -- PolyBench-shaped rank-1 structure scaled to the paper's Table 4
  "Default" value range:  X[i][j] = ((i*j) / ((R-1)(C-1))) * hi,
  v[i] = (i / (n-1)) * hi, evaluated in fp64 then rounded (RNE, numpy cast) to fp32.
* ``random`` -- the paper's Random set, values in 0.0-1.0:
  u = (splitmix64(seed_m + i) >> 11) * 2^-53, seed_m = 20200222 + 1000003*m + seed.
* ``image``  -- substitute for the Image set (ILSVRC 0-256; the dataset
  is out of scope): floor(256 u), integers 0..255 (exact in fp16).

Objects are described by the caller (``rows``, ``cols``, ``role`` per object,
from either side's object table) so this module carries no app definitions.
"""
from __future__ import annotations

import math

import numpy as np

# Table 4 "Default" upper range per app; per-object overrides.
DEFAULT_HI = {
    "gemm": 513.0, "2mm": 2051.0, "3mm": 515.0, "atax": 4094.0,
    "bicg": 4096.0, "gesummv": 4096.0, "corr": 2047.0, "covar": 2048.0,
    "mvt": 2.0, "syrk": 1026.0, "conv2d": 1.0, "syr2k": 2050.0, "conv3d": 59.0, "fdtd2d": 2041.0,
}
# BICG's r and p vectors span 0 - 4096*pi (Table 4)
DEFAULT_HI_OBJECT = {("bicg", "r"): 4096.0 * math.pi, ("bicg", "p"): 4096.0 * math.pi}

SEED_BASE = 20200222
SEED_STRIDE = 1000003
_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Counter-based splitmix64 on a uint64 array (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def uniform01(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """u_i = (splitmix64(seed + offset + i) >> 11) * 2^-53, exactly in fp64."""
    idx = np.arange(offset, offset + n, dtype=np.uint64) + np.uint64(seed & 0xFFFFFFFFFFFFFFFF)
    return (splitmix64(idx) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def default_values(rows: int, cols: int, hi: float) -> np.ndarray:
    if rows == 1:                      # vector: v[i] = (i / (n-1)) * hi
        n = cols
        i = np.arange(n, dtype=np.float64)
        return ((i / float(max(n - 1, 1))) * hi).reshape(1, n)
    denom = float(max(rows - 1, 1) * max(cols - 1, 1))
    i = np.arange(rows, dtype=np.int64)
    j = np.arange(cols, dtype=np.int64)
    return (np.outer(i, j).astype(np.float64) / denom) * hi


def object_values(kind: str, m: int, name: str, rows: int, cols: int,
                  input_set: str = "default", seed: int = 0) -> np.ndarray:
    """fp32 contents (rows x cols) of input object number m."""
    if input_set == "default":
        hi = DEFAULT_HI_OBJECT.get((kind, name), DEFAULT_HI[kind])
        v = default_values(rows, cols, hi)
    elif input_set in ("random", "image"):
        u = uniform01(SEED_BASE + SEED_STRIDE * m + seed, rows * cols).reshape(rows, cols)
        v = u if input_set == "random" else np.floor(256.0 * u)
    else:
        raise ValueError("unknown input set %r" % input_set)
    return v.astype(np.float32)


def make_inputs(kind: str, objects, input_set: str = "default", seed: int = 0) -> list:
    """One fp32 array per object with role in (0) or inout (2); None otherwise.

    ``objects``: sequence of dicts/objects with ``name``, ``rows``, ``cols``, ``role``.
    """
    out = []
    for m, o in enumerate(objects):
        get = (lambda k: o[k]) if isinstance(o, dict) else (lambda k: getattr(o, k))
        if get("role") in (0, 2):
            out.append(object_values(kind, m, get("name"), int(get("rows")), int(get("cols")),
                                     input_set, seed))
        else:
            out.append(None)
    return out
