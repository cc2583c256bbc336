"""Thin ctypes binding of libprescaler.so (include/prescaler.h).

Argument marshalling only: every step of the hot path runs in the CUDA kernels
behind the C ABI.  PyTorch provides device memory and streams.  There is no
CPU fallback: if the shared library is missing or fails to load, every call
raises ``PsError``.
"""
from __future__ import annotations

import ctypes
import os
import threading

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libprescaler.so")

F64, F32, F16 = 0, 1, 2                      # ps_dtype (descending precision)
BF16 = 3                                     # Blackwell extension (reading #28)
E4M3, E5M2 = 4, 5                            # fp8 objects with a per-tensor scale (reading #29)
METRIC_MRE, METRIC_MAX_REL = 0, 1
FLAG_NO_TENSOR_CORES = 1
FLAG_BF16 = 2                                # configuration alphabet {f64, f32, f16, bf16}: 4^M
FLAG_FP8 = 4                                 # + e4m3, e5m2: 6^M (set before bind)
ROLE_IN, ROLE_OUT, ROLE_INOUT, ROLE_TEMP = 0, 1, 2, 3

# every symbol include/prescaler.h declares
SYMBOLS = [
    "ps_status_string", "ps_last_error", "ps_version", "ps_kernel_launches", "ps_f64_uses_dmma",
    "ps_convert",
    "ps_convert_scaled", "ps_quality",
    "ps_app_create", "ps_app_destroy", "ps_app_num_objects", "ps_app_object_info",
    "ps_app_set_flags", "ps_app_workspace_bytes", "ps_app_bind", "ps_app_load_host",
    "ps_app_reference", "ps_app_set_reference", "ps_config_encode", "ps_config_decode",
    "ps_run_config", "ps_sweep", "ps_search", "ps_host_convert", "ps_run_config_host",
    "ps_transfer", "ps_app_shard_rows", "ps_app_shard_triangular", "ps_app_reference_rows",
    "ps_app_reference_merge", "ps_app_eval_shard_rows", "ps_shard_bounds", "ps_shard_step",
]
# type-conversion methods for host inputs (Fig. 3)
XFER_DEVICE, XFER_HOST_LOOP, XFER_HOST_SIMD, XFER_PIPELINE, XFER_TRANSIENT = 0, 1, 2, 3, 4


class PsError(RuntimeError):
    pass


class PsQualityResult(ctypes.Structure):
    _fields_ = [("quality", ctypes.c_double), ("mean_rel", ctypes.c_double),
                ("max_rel", ctypes.c_double), ("n", ctypes.c_uint64),
                ("nonfinite", ctypes.c_uint64)]


class PsObjectInfo(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char_p), ("n", ctypes.c_uint64), ("rows", ctypes.c_int64),
                ("cols", ctypes.c_int64), ("orig", ctypes.c_int32), ("role", ctypes.c_int32),
                ("is_output", ctypes.c_int32), ("reserved", ctypes.c_int32)]


class PsResult(ctypes.Structure):
    _fields_ = [("config_id", ctypes.c_uint64), ("convert_ms", ctypes.c_float),
                ("kernel_ms", ctypes.c_float), ("backconv_ms", ctypes.c_float),
                ("quality_ms", ctypes.c_float), ("total_ms", ctypes.c_float),
                ("transfer_ms", ctypes.c_float), ("quality", ctypes.c_double),
                ("max_rel", ctypes.c_double), ("nonfinite", ctypes.c_uint64),
                ("pass_", ctypes.c_int32), ("status", ctypes.c_int32)]


class PsShardRegion(ctypes.Structure):
    _fields_ = [("ptr", ctypes.c_void_p), ("off", ctypes.c_uint64), ("len", ctypes.c_uint64)]


class PsShardStep(ctypes.Structure):
    _fields_ = [("done", ctypes.c_int32), ("nregions", ctypes.c_int32), ("region", PsShardRegion * 4),
                ("result", PsResult)]


class PsSearchResult(ctypes.Structure):
    _fields_ = [("config_id", ctypes.c_uint64), ("total_ms", ctypes.c_float),
                ("pfp_ms", ctypes.c_float), ("quality", ctypes.c_double), ("pass_", ctypes.c_int32),
                ("trials", ctypes.c_int32), ("pfp_id", ctypes.c_uint64),
                ("trial_ids", ctypes.c_uint64 * 64), ("trial_ms", ctypes.c_float * 64),
                ("trial_pass", ctypes.c_int32 * 64)]


RESULT_DTYPE = np.dtype([("config_id", "<u8"), ("convert_ms", "<f4"), ("kernel_ms", "<f4"),
                         ("backconv_ms", "<f4"), ("quality_ms", "<f4"), ("total_ms", "<f4"),
                         ("transfer_ms", "<f4"), ("quality", "<f8"), ("max_rel", "<f8"),
                         ("nonfinite", "<u8"), ("pass", "<i4"), ("status", "<i4")])
assert ctypes.sizeof(PsResult) == 64 and RESULT_DTYPE.itemsize == 64

_lock = threading.Lock()
_lib = None
vp, i64p = ctypes.c_void_p, ctypes.POINTER(ctypes.c_int64)


def lib():
    """Load libprescaler.so (raises PsError if it is missing: no fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise PsError("libprescaler.so not built (run __graft_entry__.build() or "
                              "python -m paper_conf_cgo_kangcp20_b200.build): " + LIB_PATH)
            L = ctypes.CDLL(LIB_PATH)
            sig = {
                "ps_status_string": (ctypes.c_char_p, [ctypes.c_int]),
                "ps_last_error": (ctypes.c_char_p, []),
                "ps_version": (ctypes.c_char_p, []),
                "ps_kernel_launches": (ctypes.c_uint64, []),
                "ps_f64_uses_dmma": (ctypes.c_int, []),
                "ps_convert": (ctypes.c_int, [vp, ctypes.c_int, vp, ctypes.c_int, ctypes.c_size_t, vp]),
                "ps_convert_scaled": (ctypes.c_int, [vp, ctypes.c_int, vp, ctypes.c_int, ctypes.c_size_t,
                                                     vp, vp]),
                "ps_quality": (ctypes.c_int, [vp, ctypes.c_int, vp, ctypes.c_size_t, ctypes.c_int, vp,
                                              ctypes.POINTER(PsQualityResult)]),
                "ps_app_create": (ctypes.c_int, [ctypes.c_char_p, i64p, ctypes.c_int,
                                                 ctypes.POINTER(ctypes.c_double), ctypes.POINTER(vp)]),
                "ps_app_destroy": (ctypes.c_int, [vp]),
                "ps_app_num_objects": (ctypes.c_int, [vp]),
                "ps_app_object_info": (ctypes.c_int, [vp, ctypes.c_int, ctypes.POINTER(PsObjectInfo)]),
                "ps_app_set_flags": (ctypes.c_int, [vp, ctypes.c_uint32]),
                "ps_app_workspace_bytes": (ctypes.c_size_t, [vp]),
                "ps_app_bind": (ctypes.c_int, [vp, vp, ctypes.c_size_t, ctypes.POINTER(vp),
                                               ctypes.POINTER(vp)]),
                "ps_app_load_host": (ctypes.c_int, [vp, ctypes.POINTER(vp), vp]),
                "ps_app_reference": (ctypes.c_int, [vp, ctypes.POINTER(vp), vp]),
                "ps_app_set_reference": (ctypes.c_int, [vp, ctypes.POINTER(vp)]),
                "ps_app_shard_rows": (ctypes.c_int64, [vp]),
                "ps_app_shard_triangular": (ctypes.c_int, [vp]),
                "ps_app_reference_rows": (ctypes.c_int, [vp, ctypes.c_int64, ctypes.c_int64,
                                                         ctypes.POINTER(vp), vp]),
                "ps_app_reference_merge": (ctypes.c_int, [vp, ctypes.POINTER(vp), vp]),
                "ps_app_eval_shard_rows": (ctypes.c_int64, [vp]),
                "ps_shard_bounds": (ctypes.c_int, [vp, ctypes.c_int, ctypes.c_int, i64p, i64p]),
                "ps_shard_step": (ctypes.c_int, [vp, ctypes.POINTER(ctypes.c_int), ctypes.c_double,
                                                 ctypes.c_int, ctypes.c_int, ctypes.c_int, vp,
                                                 ctypes.POINTER(PsShardStep)]),
                "ps_config_encode": (ctypes.c_int, [vp, ctypes.POINTER(ctypes.c_int),
                                                    ctypes.POINTER(ctypes.c_uint64)]),
                "ps_config_decode": (ctypes.c_int, [vp, ctypes.c_uint64, ctypes.POINTER(ctypes.c_int)]),
                "ps_run_config": (ctypes.c_int, [vp, ctypes.POINTER(ctypes.c_int), ctypes.c_double, vp,
                                                 ctypes.POINTER(PsResult)]),
                "ps_sweep": (ctypes.c_int, [vp, ctypes.POINTER(ctypes.c_uint64), ctypes.c_size_t,
                                            ctypes.c_double, vp, ctypes.POINTER(PsResult), i64p]),
                "ps_search": (ctypes.c_int, [vp, ctypes.c_double, ctypes.c_int, vp,
                                             ctypes.POINTER(PsSearchResult)]),
                "ps_host_convert": (ctypes.c_int, [vp, vp, ctypes.c_int, ctypes.c_size_t, ctypes.c_int,
                                                   ctypes.c_int]),
                "ps_transfer": (ctypes.c_int, [vp, vp, ctypes.c_int, ctypes.c_size_t, ctypes.c_int,
                                               ctypes.c_int, vp, vp, ctypes.POINTER(ctypes.c_float)]),
                "ps_run_config_host": (ctypes.c_int, [vp, ctypes.POINTER(ctypes.c_int),
                                                      ctypes.POINTER(ctypes.c_int), ctypes.POINTER(vp),
                                                      ctypes.POINTER(vp), ctypes.c_int, ctypes.c_double,
                                                      vp, ctypes.POINTER(PsResult)]),
            }
            for name, (res, args) in sig.items():
                f = getattr(L, name)
                f.restype, f.argtypes = res, args
            _lib = L
    return _lib


def ps_status_string(s: int) -> str:
    return lib().ps_status_string(s).decode()


def ps_last_error() -> str:
    return lib().ps_last_error().decode()


def ps_version() -> str:
    return lib().ps_version().decode()


def ps_kernel_launches() -> int:
    return int(lib().ps_kernel_launches())


def _check(status: int, what: str):
    if status != 0:
        raise PsError("%s: %s (%s)" % (what, ps_status_string(status), ps_last_error()))


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def torch_dtype(code: int):
    import torch
    return {F64: torch.float64, F32: torch.float32, F16: torch.float16, BF16: torch.bfloat16,
            E4M3: torch.uint8, E5M2: torch.uint8}[code]


# -------------------------------------------------------------- (1) convert
def ps_convert(src, src_type: int, dst, dst_type: int, n: int = None, stream=None) -> None:
    """dst[i] = RNE_{dst_type}(src[i]), asynchronous on `stream` (device pointers/tensors)."""
    if n is None:
        n = src.numel()
    _check(lib().ps_convert(_ptr(src), src_type, _ptr(dst), dst_type, n, _stream(stream)),
           "ps_convert")


def ps_convert_scaled(src, src_type: int, dst, dst_type: int, scale, n: int = None,
                      stream=None) -> None:
    """fp8 object conversion with a per-tensor power-of-two scale (reading #29).
    scale: a 16-byte device buffer (ps_fp8_scale: u64 amax bits, i32 k, i32 pad);
    to fp8 it receives k, from fp8 it supplies k."""
    if n is None:
        n = src.numel()
    _check(lib().ps_convert_scaled(_ptr(src), src_type, _ptr(dst), dst_type, n, _ptr(scale),
                                   _stream(stream)), "ps_convert_scaled")


def ps_host_convert(src: np.ndarray, dst_type: int, threads: int = 0, simd: bool = True) -> np.ndarray:
    """Host-side RNE conversion of an f32 numpy array (Fig. 3a: simd=False, threads=1;
    Fig. 3b: SIMD + threads).  Bit-identical to ps_convert."""
    src = np.ascontiguousarray(src, dtype=np.float32)
    out = np.empty(src.shape, dtype={F64: np.float64, F32: np.float32, F16: np.float16,
                                     BF16: np.uint16}[dst_type])
    _check(lib().ps_host_convert(src.ctypes.data, out.ctypes.data, dst_type, src.size, threads,
                                 1 if simd else 0), "ps_host_convert")
    return out


def ps_transfer(host_src, dev_dst, dst_type: int, n: int, method: int, threads: int = 0,
                dev_stage=None, stream=None) -> float:
    """One object's {conversion then transfer} with a Fig. 3 method; returns ms."""
    ms = ctypes.c_float(0.0)
    _check(lib().ps_transfer(_ptr(host_src), _ptr(dev_dst), dst_type, n, method, threads,
                             _ptr(dev_stage), _stream(stream), ctypes.byref(ms)), "ps_transfer")
    return float(ms.value)


# -------------------------------------------------------------- (2) quality
def ps_quality(out, out_type: int, ref, n: int = None, metric: int = METRIC_MRE,
               stream=None) -> dict:
    if n is None:
        n = out.numel()
    r = PsQualityResult()
    _check(lib().ps_quality(_ptr(out), out_type, _ptr(ref), n, metric, _stream(stream),
                            ctypes.byref(r)), "ps_quality")
    return {k: getattr(r, k) for k, _ in r._fields_}


# ------------------------------------------------------- (3)-(5) apps
class App:
    """One ps_app handle: memory objects + statements of a PolyBench-shaped app."""

    def __init__(self, kind: str, dims, scalars=None):
        dims = [int(d) for d in (dims if hasattr(dims, "__len__") else [dims])]
        self.kind, self.dims = kind, dims
        d = (ctypes.c_int64 * len(dims))(*dims)
        sc = None if scalars is None else (ctypes.c_double * len(scalars))(*map(float, scalars))
        h = vp()
        _check(lib().ps_app_create(kind.encode(), d, len(dims), sc, ctypes.byref(h)), "ps_app_create")
        self._h = h
        self.num_objects = lib().ps_app_num_objects(h)
        self.objects = []
        for m in range(self.num_objects):
            info = PsObjectInfo()
            _check(lib().ps_app_object_info(h, m, ctypes.byref(info)), "ps_app_object_info")
            self.objects.append(dict(name=info.name.decode(), n=info.n, rows=info.rows,
                                     cols=info.cols, orig=info.orig, role=info.role,
                                     is_output=bool(info.is_output)))
        self.workspace_bytes = int(lib().ps_app_workspace_bytes(h))
        self.flags = 0
        self._keep = []
        self.inputs = self.outputs = self.ref = None

    def close(self):
        if getattr(self, "_h", None):
            lib().ps_app_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def radix(self) -> int:
        return 6 if self.flags & FLAG_FP8 else (4 if self.flags & FLAG_BF16 else 3)

    @property
    def space(self) -> int:
        return self.radix ** self.num_objects

    def set_flags(self, flags: int):
        """PS_FLAG_* bits; FLAG_FP8 changes the workspace size, so set it before bind()."""
        _check(lib().ps_app_set_flags(self._h, flags), "ps_app_set_flags")
        self.flags = int(flags)
        self.workspace_bytes = int(lib().ps_app_workspace_bytes(self._h))

    def bind(self, inputs, outputs=None, workspace=None, device=None):
        """inputs: per object an f32 CUDA tensor (role in/inout) or None.
        outputs/workspace are allocated with torch when not given."""
        import torch
        dev = device or next(t.device for t in inputs if t is not None)
        if outputs is None:
            outputs = [torch.empty(o["n"], dtype=torch.float32, device=dev) if o["is_output"] else None
                       for o in self.objects]
        if workspace is None:
            workspace = torch.empty(self.workspace_bytes, dtype=torch.uint8, device=dev)
        ins = (vp * self.num_objects)(*[_ptr(t) for t in inputs])
        outs = (vp * self.num_objects)(*[_ptr(t) for t in outputs])
        _check(lib().ps_app_bind(self._h, _ptr(workspace), self.workspace_bytes, ins, outs),
               "ps_app_bind")
        self.inputs, self.outputs, self.workspace = list(inputs), outputs, workspace
        return outputs

    def load_host(self, host_inputs, stream=None):
        arr = (vp * self.num_objects)(*[_ptr(t) if t is not None else None for t in host_inputs])
        _check(lib().ps_app_load_host(self._h, arr, _stream(stream)), "ps_app_load_host")

    def reference(self, stream=None, refs=None):
        """a0: the all-f64 run; fills (or allocates) one fp64 buffer per output object."""
        import torch
        dev = self.workspace.device
        if refs is None:
            refs = [torch.empty(o["n"], dtype=torch.float64, device=dev) if o["is_output"] else None
                    for o in self.objects]
        arr = (vp * self.num_objects)(*[_ptr(t) for t in refs])
        _check(lib().ps_app_reference(self._h, arr, _stream(stream)), "ps_app_reference")
        self.ref = refs
        return refs

    @property
    def shard_rows(self) -> int:
        """Rows of the output a reference shard computes (0: not row-shardable)."""
        return int(lib().ps_app_shard_rows(self._h))

    @property
    def shard_triangular(self) -> bool:
        return bool(lib().ps_app_shard_triangular(self._h))

    def alloc_refs(self):
        import torch
        dev = self.workspace.device
        return [torch.empty(o["n"], dtype=torch.float64, device=dev) if o["is_output"] else None
                for o in self.objects]

    def reference_rows(self, row0: int, row1: int, refs, stream=None):
        """ps_app_reference_rows: rows [row0, row1) of the fp64 reference into refs."""
        arr = (vp * self.num_objects)(*[_ptr(t) for t in refs])
        _check(lib().ps_app_reference_rows(self._h, int(row0), int(row1), arr, _stream(stream)),
               "ps_app_reference_rows")
        return refs

    def reference_merge(self, refs, stream=None):
        """ps_app_reference_merge: mirror (triangular outputs) and adopt refs."""
        arr = (vp * self.num_objects)(*[_ptr(t) for t in refs])
        _check(lib().ps_app_reference_merge(self._h, arr, _stream(stream)), "ps_app_reference_merge")
        self.ref = list(refs)
        return refs

    # ------------------------------------------- row-sharded evaluation (4b)
    @property
    def eval_shard_rows(self) -> int:
        """Rows of the dimension a row-sharded evaluation splits (0: not supported)."""
        return int(lib().ps_app_eval_shard_rows(self._h))

    def shard_bounds(self, rank: int, world: int):
        r0, r1 = ctypes.c_int64(), ctypes.c_int64()
        _check(lib().ps_shard_bounds(self._h, int(rank), int(world), ctypes.byref(r0), ctypes.byref(r1)),
               "ps_shard_bounds")
        return int(r0.value), int(r1.value)

    def shard_step(self, prec, rank: int, world: int, stage: int, toq: float = 0.9, stream=None):
        """One stage of the row-sharded evaluation.  Returns (done, regions, result):
        regions = [(workspace byte offset of the buffer, off, len)] to exchange, result
        the record once done."""
        p = (ctypes.c_int * self.num_objects)(*prec)
        x = PsShardStep()
        _check(lib().ps_shard_step(self._h, p, float(toq), int(rank), int(world), int(stage),
                                   _stream(stream), ctypes.byref(x)), "ps_shard_step")
        base = self.workspace.data_ptr()
        regions = [(int(x.region[k].ptr) - base, int(x.region[k].off), int(x.region[k].len))
                   for k in range(x.nregions)]
        res = _result_dict(np.frombuffer(bytes(x.result), dtype=RESULT_DTYPE)[0]) if x.done else None
        return bool(x.done), regions, res

    def set_reference(self, refs):
        arr = (vp * self.num_objects)(*[_ptr(t) for t in refs])
        _check(lib().ps_app_set_reference(self._h, arr), "ps_app_set_reference")
        self.ref = list(refs)

    def encode(self, prec) -> int:
        p = (ctypes.c_int * self.num_objects)(*prec)
        out = ctypes.c_uint64()
        _check(lib().ps_config_encode(self._h, p, ctypes.byref(out)), "ps_config_encode")
        return int(out.value)

    def decode(self, cid: int) -> list:
        p = (ctypes.c_int * self.num_objects)()
        _check(lib().ps_config_decode(self._h, int(cid), p), "ps_config_decode")
        return list(p)

    def run_config(self, prec, toq: float = 0.9, stream=None, sync: bool = True):
        p = (ctypes.c_int * self.num_objects)(*prec)
        r = PsResult() if sync else None
        _check(lib().ps_run_config(self._h, p, float(toq), _stream(stream),
                                   ctypes.byref(r) if sync else None), "ps_run_config")
        if not sync:
            return None
        return _result_dict(np.frombuffer(bytes(r), dtype=RESULT_DTYPE)[0])

    def sweep_raw(self, config_ids, toq: float = 0.9, stream=None):
        """ps_sweep -> (numpy structured array of ps_result, best index)."""
        ids = np.ascontiguousarray(np.asarray(config_ids, dtype=np.uint64))
        res = (PsResult * max(len(ids), 1))()
        best = ctypes.c_int64(-1)
        _check(lib().ps_sweep(self._h, ids.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)),
                              len(ids), float(toq), _stream(stream), res, ctypes.byref(best)),
               "ps_sweep")
        arr = np.frombuffer(bytes(res), dtype=RESULT_DTYPE)[:len(ids)].copy()
        return arr, int(best.value)

    def run_config_host(self, prec, host_inputs, methods=None, host_outputs=None, threads: int = 0,
                        toq: float = 0.9, stream=None) -> dict:
        """ps_run_config_host: the configuration from host f32 inputs with per-object
        conversion methods (XFER_*); transfer_ms and total_ms include the transfers."""
        m = self.num_objects
        p = (ctypes.c_int * m)(*prec)
        meth = None if methods is None else (ctypes.c_int * m)(*methods)
        hin = (vp * m)(*[_ptr(t) if t is not None else None for t in host_inputs])
        hout = None if host_outputs is None else (vp * m)(*[_ptr(t) if t is not None else None
                                                          for t in host_outputs])
        r = PsResult()
        _check(lib().ps_run_config_host(self._h, p, meth, hin, hout, int(threads), float(toq),
                                        _stream(stream), ctypes.byref(r)), "ps_run_config_host")
        return _result_dict(np.frombuffer(bytes(r), dtype=RESULT_DTYPE)[0])

    def search(self, toq: float = 0.9, repeats: int = 1, stream=None) -> dict:
        """ps_search: PFP initialisation + Alg. 1 normal search (decision tree)."""
        r = PsSearchResult()
        _check(lib().ps_search(self._h, float(toq), int(repeats), _stream(stream), ctypes.byref(r)),
               "ps_search")
        return {"config_id": int(r.config_id), "prec": self.decode(r.config_id),
                "total_ms": float(r.total_ms), "quality": float(r.quality), "pass": bool(r.pass_),
                "trials": int(r.trials), "pfp_id": int(r.pfp_id), "pfp_ms": float(r.pfp_ms),
                "trial_ids": [int(x) for x in r.trial_ids[:min(r.trials, 64)]],
                "trial_ms": [float(x) for x in r.trial_ms[:min(r.trials, 64)]],
                "trial_pass": [bool(x) for x in r.trial_pass[:min(r.trials, 64)]]}

    def sweep(self, config_ids, toq: float = 0.9, stream=None):
        arr, best = self.sweep_raw(config_ids, toq, stream)
        return [_result_dict(r) for r in arr], best


def _result_dict(r) -> dict:
    d = {k: r[k].item() for k in RESULT_DTYPE.names if k != "reserved"}
    d["pass"] = bool(d["pass"])
    return d
