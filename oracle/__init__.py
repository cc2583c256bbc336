"""PreScaler CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` leg may import this package.  The product path
(``paper_conf_cgo_kangcp20_b200``) never imports it and shares no code with it.

This module is argument marshalling (ctypes + numpy) around ``oracle.c``, the
plain single-threaded C definition of SURVEY.md §8(a) a1-a5 (see the header of
``oracle.c`` for the paper passages each part follows).  Precision codes:
0 = f64, 1 = f32, 2 = f16 (descending precision); 3 = bf16 for the
Blackwell extension, whose buffers are raw uint16 bit
patterns here (numpy has no bfloat16; ``widen`` gives their exact values);
4 = fp8 E4M3 and 5 = fp8 E5M2 (reading #29), raw uint8 codes whose objects
carry a per-tensor power-of-two scale 2^k (``convert_scaled``,
``run_config(..., with_scales=True)``).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-std=c11", "-Wall"]

F64, F32, F16, BF16, E4M3, E5M2 = 0, 1, 2, 3, 4, 5
NP_DTYPE = {F64: np.float64, F32: np.float32, F16: np.float16, BF16: np.uint16,
            E4M3: np.uint8, E5M2: np.uint8}
FP8 = (E4M3, E5M2)
FP8_MAX = {E4M3: 448.0, E5M2: 57344.0}
ROWDOT_LANES = 32
COLSUM_CHUNK = 256

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so (gcc, no fast-math, no FMA contraction)."""
    stale = (not os.path.exists(_LIB)) or os.path.getmtime(_LIB) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h")))
    if force or stale:
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class QualityResult(ctypes.Structure):
    _fields_ = [("quality", ctypes.c_double), ("mean_rel", ctypes.c_double),
                ("max_rel", ctypes.c_double), ("n", ctypes.c_uint64),
                ("nonfinite", ctypes.c_uint64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class ObjectInfo(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char_p), ("role", ctypes.c_int), ("is_output", ctypes.c_int),
                ("rows", ctypes.c_int64), ("cols", ctypes.c_int64)]


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = ctypes.CDLL(build())
            L.oracle_convert_bits.restype = ctypes.c_uint64
            L.oracle_convert_bits.argtypes = [ctypes.c_uint64, ctypes.c_int, ctypes.c_int]
            L.oracle_convert.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p,
                                         ctypes.c_int, ctypes.c_size_t]
            L.oracle_quality.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p,
                                         ctypes.c_size_t, ctypes.POINTER(QualityResult)]
            L.oracle_fp8_scale_exp.argtypes = [ctypes.c_double, ctypes.c_int]
            L.oracle_convert_scaled.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p,
                                                ctypes.c_int, ctypes.c_size_t,
                                                ctypes.POINTER(ctypes.c_int)]
            L.oracle_run_config_k.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_int64),
                                              ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                                              ctypes.POINTER(ctypes.c_int),
                                              ctypes.POINTER(ctypes.c_void_p),
                                              ctypes.POINTER(ctypes.c_void_p),
                                              ctypes.POINTER(ctypes.c_int)]
            L.oracle_config_decode.argtypes = [ctypes.c_int, ctypes.c_uint64,
                                               ctypes.POINTER(ctypes.c_int)]
            L.oracle_config_encode.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_int),
                                               ctypes.POINTER(ctypes.c_uint64)]
            L.oracle_config_decode_radix.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_uint64,
                                                     ctypes.POINTER(ctypes.c_int)]
            L.oracle_config_encode_radix.argtypes = [ctypes.c_int, ctypes.c_int,
                                                     ctypes.POINTER(ctypes.c_int),
                                                     ctypes.POINTER(ctypes.c_uint64)]
            L.oracle_app_objects.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_int64),
                                             ctypes.c_int, ctypes.POINTER(ObjectInfo)]
            L.oracle_run_config.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_int64),
                                            ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                                            ctypes.POINTER(ctypes.c_int),
                                            ctypes.POINTER(ctypes.c_void_p),
                                            ctypes.POINTER(ctypes.c_void_p)]
            L.oracle_evaluate.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_int64),
                                          ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                                          ctypes.POINTER(ctypes.c_int),
                                          ctypes.POINTER(ctypes.c_void_p),
                                          ctypes.POINTER(ctypes.c_void_p),
                                          ctypes.POINTER(ctypes.c_void_p),
                                          ctypes.POINTER(QualityResult)]
            _lib = L
    return _lib


def _ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


# ---------------------------------------------------------------- conversion
def convert_bits(bits: int, src: int, dst: int) -> int:
    return int(lib().oracle_convert_bits(bits, src, dst))


def convert(a: np.ndarray, src: int, dst: int) -> np.ndarray:
    """Element-wise RNE conversion with the software converter (c-1)."""
    a = np.ascontiguousarray(a)
    assert a.dtype == NP_DTYPE[src] or a.dtype.itemsize == np.dtype(NP_DTYPE[src]).itemsize
    out = np.empty(a.shape, dtype=NP_DTYPE[dst])
    if lib().oracle_convert(_ptr(a), src, _ptr(out), dst, a.size):
        raise ValueError("oracle_convert failed")
    return out


def fp8_scale_exp(amax: float, t: int) -> int:
    """Reading #29: smallest k in [-126, 126] with amax <= FMAX * 2^k."""
    return int(lib().oracle_fp8_scale_exp(float(amax), t))


def convert_scaled(a: np.ndarray, src: int, dst: int, k: int = 0):
    """Scaled conversion (reading #29).  To fp8: returns (codes, k) with k from
    the finite values of a.  From fp8: returns (values, k) decoding with scale 2^k."""
    a = np.ascontiguousarray(a)
    out = np.empty(a.shape, dtype=NP_DTYPE[dst])
    kk = ctypes.c_int(int(k))
    if lib().oracle_convert_scaled(_ptr(a), src, _ptr(out), dst, a.size, ctypes.byref(kk)):
        raise ValueError("oracle_convert_scaled failed")
    return out, int(kk.value)


def widen(a: np.ndarray, t: int) -> np.ndarray:
    """Exact float64 values of a buffer stored in precision t (bf16: raw uint16)."""
    a = np.ascontiguousarray(a)
    if t == F64:
        return a.astype(np.float64)
    return convert(a, t, F64)


# ------------------------------------------------------------------- quality
def quality(out: np.ndarray, out_type: int, ref: np.ndarray) -> dict:
    out = np.ascontiguousarray(out)
    ref = np.ascontiguousarray(ref, dtype=np.float64)
    assert out.size == ref.size
    r = QualityResult()
    if lib().oracle_quality(_ptr(out), out_type, _ptr(ref), out.size, ctypes.byref(r)):
        raise ValueError("oracle_quality failed")
    return r.as_dict()


# --------------------------------------------------------------------- codec
def config_decode(num_objects: int, cid: int, radix: int = 3) -> list:
    p = (ctypes.c_int * num_objects)()
    if lib().oracle_config_decode_radix(num_objects, radix, cid, p):
        raise ValueError("bad config id")
    return list(p)


def config_encode(prec, radix: int = 3) -> int:
    p = (ctypes.c_int * len(prec))(*prec)
    out = ctypes.c_uint64()
    if lib().oracle_config_encode_radix(len(prec), radix, p, ctypes.byref(out)):
        raise ValueError("bad precision vector")
    return int(out.value)


# ---------------------------------------------------------------------- apps
def _dims(dims):
    dims = [int(d) for d in (dims if hasattr(dims, "__len__") else [dims])]
    return (ctypes.c_int64 * len(dims))(*dims), len(dims)


def app_objects(kind: str, dims) -> list:
    d, nd = _dims(dims)
    info = (ObjectInfo * 8)()
    n = lib().oracle_app_objects(kind.encode(), d, nd, info)
    if n < 0:
        raise ValueError("unknown app or bad dims: %s %s" % (kind, dims))
    return [dict(name=info[m].name.decode(), role=info[m].role, is_output=bool(info[m].is_output),
                 rows=info[m].rows, cols=info[m].cols) for m in range(n)]


def _scalars(scalars):
    if scalars is None:
        return None
    return (ctypes.c_double * len(scalars))(*[float(s) for s in scalars])


def _inputs(objs, inputs):
    keep, arr = [], (ctypes.c_void_p * len(objs))()
    for m, o in enumerate(objs):
        if o["role"] in (0, 2):
            a = np.ascontiguousarray(inputs[m], dtype=np.float32).reshape(-1)
            assert a.size == o["rows"] * o["cols"], (o, a.size)
            keep.append(a)
            arr[m] = a.ctypes.data
    return arr, keep


def run_config(kind: str, dims, prec, inputs, scalars=None, with_scales: bool = False):
    """a2 + a3: final contents of every object in its assigned precision (fp8:
    raw codes).  with_scales: also return the list of final scale exponents k
    (None for non-fp8 objects)."""
    objs = app_objects(kind, dims)
    assert len(prec) == len(objs)
    d, nd = _dims(dims)
    ins, keep = _inputs(objs, inputs)
    finals = [np.empty((o["rows"], o["cols"]), dtype=NP_DTYPE[p]) for o, p in zip(objs, prec)]
    fin = (ctypes.c_void_p * len(objs))(*[f.ctypes.data for f in finals])
    pr = (ctypes.c_int * len(prec))(*prec)
    ks = (ctypes.c_int * len(prec))()
    if lib().oracle_run_config_k(kind.encode(), d, nd, _scalars(scalars), pr, ins, fin, ks):
        raise ValueError("oracle_run_config failed")
    if with_scales:
        return finals, [int(ks[m]) if p in FP8 else None for m, p in enumerate(prec)]
    return finals


def values(final: np.ndarray, t: int, k=None) -> np.ndarray:
    """Exact float64 values of an object's final contents (fp8: code * 2^k)."""
    if t in FP8:
        return np.ldexp(widen(final, t), int(k))
    return widen(final, t)


def reference(kind: str, dims, inputs, scalars=None) -> list:
    """The full-precision (all-f64) run: raw fp64 contents of every object."""
    objs = app_objects(kind, dims)
    return run_config(kind, dims, [F64] * len(objs), inputs, scalars)


def evaluate(kind: str, dims, prec, inputs, ref, scalars=None, toq: float = 0.9):
    """a2-a5 for one configuration.  ref = list per object (fp64 for outputs).
    Returns (result dict incl. 'pass', delivered f32 outputs per object or None)."""
    objs = app_objects(kind, dims)
    d, nd = _dims(dims)
    ins, keep = _inputs(objs, inputs)
    refs = (ctypes.c_void_p * len(objs))()
    dels = (ctypes.c_void_p * len(objs))()
    delivered = [None] * len(objs)
    for m, o in enumerate(objs):
        if o["is_output"]:
            r = np.ascontiguousarray(ref[m], dtype=np.float64).reshape(-1)
            keep.append(r)
            refs[m] = r.ctypes.data
            delivered[m] = np.empty((o["rows"], o["cols"]), dtype=np.float32)
            dels[m] = delivered[m].ctypes.data
    res = QualityResult()
    pr = (ctypes.c_int * len(prec))(*prec)
    if lib().oracle_evaluate(kind.encode(), d, nd, _scalars(scalars), pr, ins, refs, dels,
                             ctypes.byref(res)):
        raise ValueError("oracle_evaluate failed")
    out = res.as_dict()
    out["pass"] = bool(out["quality"] >= toq)     # Alg. 1 l.10: fail iff Accuracy < TOQ
    return out, delivered


def sample(kind: str, dims, prec, inputs, m: int, rows, cols, scalars=None) -> np.ndarray:
    """Raw final values (in precision prec[m], widened to float64) of output
    object m at entries (rows[k], cols[k]); only what they depend on is computed."""
    L = lib()
    if not hasattr(L, "_sample_sig"):
        L.oracle_sample.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_int64), ctypes.c_int,
                                    ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int),
                                    ctypes.POINTER(ctypes.c_void_p), ctypes.c_int,
                                    ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t,
                                    ctypes.c_void_p]
        L._sample_sig = True
    objs = app_objects(kind, dims)
    d, nd = _dims(dims)
    ins, keep = _inputs(objs, inputs)
    r = np.ascontiguousarray(rows, dtype=np.int64)
    c = np.ascontiguousarray(cols, dtype=np.int64)
    out = np.empty(r.size, dtype=np.float64)
    pr = (ctypes.c_int * len(prec))(*prec)
    if L.oracle_sample(kind.encode(), d, nd, _scalars(scalars), pr, ins, m, r.ctypes.data,
                       c.ctypes.data, r.size, out.ctypes.data):
        raise ValueError("oracle_sample failed")
    return out


def sweep(kind: str, dims, config_ids, inputs, scalars=None, toq: float = 0.9, ref=None):
    """c-6: evaluate every configuration id; returns (ref, list of result dicts)."""
    objs = app_objects(kind, dims)
    if ref is None:
        ref = reference(kind, dims, inputs, scalars)
    results = []
    for cid in config_ids:
        prec = config_decode(len(objs), cid)
        r, _ = evaluate(kind, dims, prec, inputs, ref, scalars, toq)
        r["config_id"] = int(cid)
        results.append(r)
    return ref, results
