"""The library's host-side conversion (Fig. 3a single loop / 3b multithreaded SIMD,
P:101-103; csrc/host_convert.cpp) vs the oracle's software converter: bit-exact over
all 2^32 fp32 inputs (NaN canonical on both sides), plus f32 -> f64.  Host code:
runs without a GPU."""
import concurrent.futures as cf

import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B


@pytest.fixture(scope="module")
def lib():
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    return B.lib()


def oracle_mt(x, dt, parts=8):
    out = np.empty(x.shape, dtype={0: np.float64, 1: np.float32, 2: np.float16}[dt])
    b = np.linspace(0, x.size, parts + 1).astype(np.int64)

    def run(i):
        out[b[i]:b[i + 1]] = oracle.convert(x[b[i]:b[i + 1]], 1, dt)
    with cf.ThreadPoolExecutor(parts) as ex:
        list(ex.map(run, range(parts)))
    return out


def test_f32_to_f16_all_2pow32_simd_and_single_loop(lib, oracle_lib):
    chunk = 1 << 26
    for c in range(1 << 6):
        x = np.arange(c * chunk, (c + 1) * chunk, dtype=np.uint64).astype(np.uint32).view(np.float32)
        want = oracle_mt(x, 2).view(np.uint16)
        simd = B.ps_host_convert(x, B.F16, threads=8, simd=True).view(np.uint16)
        loop = B.ps_host_convert(x, B.F16, threads=8, simd=False).view(np.uint16)
        assert np.array_equal(simd, want), c
        assert np.array_equal(loop, want), c


def test_f32_to_f64_and_copy(lib, oracle_lib):
    rng = np.random.default_rng(4)
    x = rng.integers(0, 2**32, size=1 << 22, dtype=np.uint64).astype(np.uint32).view(np.float32)
    want = oracle.convert(x, 1, 0).view(np.uint64)
    for simd in (True, False):
        got = B.ps_host_convert(x, B.F64, threads=4, simd=simd).view(np.uint64)
        assert np.array_equal(got, want)
    assert np.array_equal(B.ps_host_convert(x, B.F32).view(np.uint32), x.view(np.uint32))


def test_ragged_and_single_thread(lib, oracle_lib):
    rng = np.random.default_rng(5)
    for n in (0, 1, 7, 9, 65537):
        x = (rng.standard_normal(n) * 3e4).astype(np.float32)
        for th in (1, 3):
            got = B.ps_host_convert(x, B.F16, threads=th).view(np.uint16)
            assert np.array_equal(got, oracle.convert(x, 1, 2).view(np.uint16))
