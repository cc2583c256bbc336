"""GPU parity of ps_convert (row a2) vs the oracle's software converter: bit-exact.

NaN inputs must give the canonical NaN (reading #5), which the oracle also
produces, so NaNs are compared bit-exactly too.
"""
import concurrent.futures as cf

import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B

pytestmark = pytest.mark.gpu

NP = {0: np.float64, 1: np.float32, 2: np.float16}
RAW = {0: np.uint64, 1: np.uint32, 2: np.uint16}


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return torch


def oracle_convert_mt(x: np.ndarray, st: int, dt: int, parts: int = 8) -> np.ndarray:
    """The oracle (single-threaded C) on 8 host threads over disjoint slices."""
    out = np.empty(x.shape, dtype=NP[dt])
    bounds = np.linspace(0, x.size, parts + 1).astype(np.int64)

    def run(i):
        a, b = bounds[i], bounds[i + 1]
        out[a:b] = oracle.convert(x[a:b], st, dt)
    with cf.ThreadPoolExecutor(parts) as ex:
        list(ex.map(run, range(parts)))
    return out


def gpu_convert(torch, x: np.ndarray, st: int, dt: int, src_off=0, dst_off=0):
    src = torch.from_numpy(np.ascontiguousarray(x).view(RAW[st]).view(np.uint8)).cuda()
    n = x.size
    s_size, d_size = np.dtype(NP[st]).itemsize, np.dtype(NP[dt]).itemsize
    if src_off:
        buf = torch.zeros(src.numel() + src_off * s_size, dtype=torch.uint8, device="cuda")
        buf[src_off * s_size:] = src
        src_ptr = buf.data_ptr() + src_off * s_size
        keep = buf
    else:
        src_ptr, keep = src.data_ptr(), src
    dst = torch.zeros((n + dst_off) * d_size + 16, dtype=torch.uint8, device="cuda")
    B.ps_convert(src_ptr, st, dst.data_ptr() + dst_off * d_size, dt, n)
    torch.cuda.synchronize()
    del keep
    return dst[dst_off * d_size:(dst_off + n) * d_size].cpu().numpy().view(NP[dt])


def test_f32_to_f16_all_2pow32(torch_cuda):
    """Every one of the 2^32 fp32 bit patterns (generated on the device from an
    index, 2^28 per chunk), bit-exact vs the oracle."""
    torch = torch_cuda
    chunk = 1 << 28
    dst = torch.empty(chunk, dtype=torch.float16, device="cuda")
    for c in range(1 << 4):
        base = c * chunk
        bits = torch.arange(base, base + chunk, dtype=torch.int64, device="cuda")
        bits = (bits - (bits >= 2**31).to(torch.int64) * 2**32).to(torch.int32)
        src = bits.view(torch.float32)
        B.ps_convert(src, 1, dst, 2)
        got = dst.view(torch.int16).cpu().numpy().view(np.uint16)
        x = (np.arange(base, base + chunk, dtype=np.uint64).astype(np.uint32)).view(np.float32)
        want = oracle_convert_mt(x, 1, 2).view(np.uint16)
        bad = np.flatnonzero(got != want)
        assert bad.size == 0, "chunk %d: %d mismatches, first input %#x got %#x want %#x" % (
            c, bad.size, x.view(np.uint32)[bad[0]], got[bad[0]], want[bad[0]])


def test_f16_widen_all(torch_cuda):
    h = np.arange(65536, dtype=np.uint32).astype(np.uint16).view(np.float16)
    for dt in (0, 1):
        got = gpu_convert(torch_cuda, h, 2, dt)
        want = oracle.convert(h, 2, dt)
        assert np.array_equal(got.view(RAW[dt]), want.view(RAW[dt]))


def _f64_targets():
    lo = oracle.convert(np.arange(0x7C00, dtype=np.uint16).view(np.float16), 2, 0)
    hi = oracle.convert(np.arange(1, 0x7C01, dtype=np.uint16).view(np.float16), 2, 0)
    hi[-1] = 65536.0
    mid = lo + (hi - lo) / 2
    mb = mid.view(np.uint64)
    sets = [lo.view(np.uint64)] + [mb + np.uint64(k) for k in range(0, 5)] + \
           [mb - np.uint64(k) for k in range(1, 5)]
    t = np.concatenate(sets)
    t = np.concatenate([t, t | np.uint64(1 << 63)])
    rng = np.random.default_rng(5)
    r = rng.integers(0, 2**63, size=1 << 22, dtype=np.int64).astype(np.uint64) * np.uint64(2) + \
        rng.integers(0, 2, size=1 << 22).astype(np.uint64)
    special = np.array([0x7FF0000000000000, 0xFFF0000000000000, 0x7FF8000000000000,
                        0xFFF0000000000001, 0, 1 << 63, 1], dtype=np.uint64)
    return np.concatenate([t, r, special]).view(np.float64)


def test_f64_to_f16_targets_and_random(torch_cuda):
    x = _f64_targets()
    got = gpu_convert(torch_cuda, x, 0, 2).view(np.uint16)
    want = oracle_convert_mt(x, 0, 2).view(np.uint16)
    bad = np.flatnonzero(got != want)
    assert bad.size == 0, "%d mismatches; first %r -> %#x want %#x" % (
        bad.size, x[bad[0]], got[bad[0]], want[bad[0]])


@pytest.mark.parametrize("st,dt", [(0, 1), (1, 0), (2, 0), (1, 2), (0, 2), (2, 1)])
def test_random_bit_patterns(torch_cuda, st, dt):
    rng = np.random.default_rng(st * 7 + dt)
    nbytes = np.dtype(NP[st]).itemsize
    x = rng.integers(0, 256, size=(1 << 21) * nbytes, dtype=np.uint8).view(NP[st])
    got = gpu_convert(torch_cuda, x, st, dt)
    want = oracle_convert_mt(x, st, dt)
    assert np.array_equal(got.view(RAW[dt]), want.view(RAW[dt]))


@pytest.mark.parametrize("st,dt", [(1, 2), (0, 2), (2, 1), (0, 1), (1, 0), (2, 0), (1, 1)])
def test_unaligned_and_ragged(torch_cuda, st, dt):
    rng = np.random.default_rng(3)
    for n in [0, 1, 3, 7, 8, 9, 31, 100, 1023, 4097, 100003]:
        for so, do in [(0, 0), (1, 0), (0, 1), (3, 5), (1, 1), (7, 2)]:
            x = (rng.standard_normal(n) * 1000).astype(NP[st])
            if n == 0:
                continue
            got = gpu_convert(torch_cuda, x, st, dt, so, do)
            want = oracle.convert(x, st, dt)
            assert np.array_equal(got.view(RAW[dt]), want.view(RAW[dt])), (n, so, do)


def test_fixed_points_on_device(torch_cuda):
    import os
    here = os.path.dirname(os.path.abspath(__file__))
    code = {"f64": 0, "f32": 1, "f16": 2}
    for raw in open(os.path.join(here, "golden", "convert_fixed_points.txt")):
        f = raw.split("#")[0].split()
        if not f:
            continue
        s, d, x, e = code[f[0]], code[f[1]], int(f[2], 16), int(f[3], 16)
        arr = np.array([x], dtype=RAW[s]).view(NP[s])
        got = gpu_convert(torch_cuda, arr, s, d).view(RAW[d])[0]
        assert int(got) == e, raw


def test_large_conversion_sampled(torch_cuda):
    """A 1 GiB f32 -> f16 conversion (the bench size class), sampled vs the oracle."""
    torch = torch_cuda
    n = 1 << 28
    g = torch.Generator(device="cuda").manual_seed(0)
    src = (torch.rand(n, device="cuda", generator=g) * 70000.0 - 35000.0)
    dst = torch.empty(n, dtype=torch.float16, device="cuda")
    B.ps_convert(src, 1, dst, 2)
    torch.cuda.synchronize()
    idx = torch.randint(0, n, (1 << 20,), device="cuda", generator=g)
    x = src[idx].cpu().numpy()
    got = dst[idx].cpu().numpy().view(np.uint16)
    assert np.array_equal(got, oracle.convert(x, 1, 2).view(np.uint16))
    # the last elements (tail of the grid-stride loop)
    x = src[-4099:].cpu().numpy()
    assert np.array_equal(dst[-4099:].cpu().numpy().view(np.uint16),
                          oracle.convert(x, 1, 2).view(np.uint16))
