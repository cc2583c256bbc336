"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (ps_app_bind + ps_run_config, same kernels as ps_sweep), on outputs the
oracle computes one by one (oracle.sample).

SIMT / mat-vec statements: bit-exact on the sampled delivered outputs (and on the
fp64 reference).  Tensor-core (fp16 x fp16) statements: 2^-10 relative per
element for positive inputs (north star), reading R6.
"""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def f32_bits(x64):
    """RNE to f32 of raw values (the a4 back-conversion), via the oracle converter."""
    return oracle.convert(np.ascontiguousarray(x64, dtype=np.float64), 0, 1).view(np.uint32)


def run(torch, kind, dims, iset, configs, samples, tc_rel=None, flags=0):
    app = B.App(kind, dims)
    app.set_flags(flags)
    ins = gen.make_inputs(kind, app.objects, iset)
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    refs = app.reference()
    m_obj = len(app.objects)
    # the fp64 reference (config 0), bit-exact on the samples
    for k, (rows, cols) in samples.items():
        want = oracle.sample(kind, dims, [0] * m_obj, ins, k, rows, cols)
        got = refs[k].view(app.objects[k]["rows"], app.objects[k]["cols"])[rows, cols].cpu().numpy()
        assert np.array_equal(got.view(np.uint64), want.view(np.uint64)), (kind, "reference", k)
    for prec in configs:
        app.run_config(prec)
        torch.cuda.synchronize()
        for k, (rows, cols) in samples.items():
            o = app.objects[k]
            raw = oracle.sample(kind, dims, prec, ins, k, rows, cols)
            got = app.outputs[k].view(o["rows"], o["cols"])[rows, cols].cpu().numpy()
            exact = tc_rel is None or not tc_rel(prec)
            if exact:
                want = f32_bits(raw)
                ok = (got.view(np.uint32) == want) | (np.isnan(got) & np.isnan(raw))
                assert np.all(ok), (kind, prec, k, np.flatnonzero(~ok)[:5], got[~ok][:3], raw[~ok][:3])
            else:
                fin = np.isfinite(raw)
                assert np.array_equal(np.isfinite(got), fin), (kind, prec, k)
                rel = np.abs(got[fin] - raw[fin]) / np.maximum(np.abs(raw[fin]), 1e-300)
                assert np.all(rel <= 2.0 ** -10), (kind, prec, k, rel.max())


def _vec_samples(n, rng, cnt=256):
    idx = np.sort(rng.choice(n, size=cnt, replace=False))
    return np.zeros(cnt, dtype=np.int64), idx


def _tc_chain(prec):
    # a statement with two fp16 multiplicands and f32 compute type exists
    return any(p == 2 for p in prec)


def _tile_rows(n, rng, count):
    """`count` distinct rows: one in each 256-row tile-row (the tcgen05 2-CTA tile), the
    rest random -- so a bug confined to some tiles of the persistent scheduler shows."""
    per = [int(t * 256 + rng.integers(0, 256)) for t in range(n // 256)]
    per = list(rng.choice(per, size=min(count, len(per)), replace=False))
    rest = [r for r in rng.permutation(n) if r not in per][:max(0, count - len(per))]
    return np.sort(np.array(per + rest, dtype=np.int64))


def run_rows(torch, kind, dims, iset, configs, m, rows, cols, tc_check=None, flags=0):
    """Delivered output m at the grid rows x cols (full rows when cols is every column)
    for each configuration, against oracle.sample; the oracle runs for all configurations
    concurrently on the host (ctypes releases the GIL) while the GPU runs."""
    from concurrent.futures import ThreadPoolExecutor
    app = B.App(kind, dims)
    app.set_flags(flags)
    ins = gen.make_inputs(kind, app.objects, iset)
    rr, cc = np.meshgrid(rows, cols, indexing="ij")
    rr, cc = rr.reshape(-1), cc.reshape(-1)
    M = app.num_objects
    with ThreadPoolExecutor(len(configs)) as ex:
        futs = [ex.submit(oracle.sample, kind, dims, p, ins, m, rr, cc) for p in configs]
        app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
        refs = app.reference()
        o = app.objects[m]
        got_ref = refs[m].view(o["rows"], o["cols"])[rr, cc].cpu().numpy()
        outs = []
        for prec in configs:
            app.run_config(prec)
            torch.cuda.synchronize()
            outs.append(app.outputs[m].view(o["rows"], o["cols"])[rr, cc].cpu().numpy())
        raws = [f.result() for f in futs]
    for prec, got, raw in zip(configs, outs, raws):
        if prec == [0] * M:   # the fp64 reference (a0) is the all-f64 run, bit for bit
            assert np.array_equal(got_ref.view(np.uint64), raw.view(np.uint64)), (kind, "reference")
        if tc_check is None or not _tc_chain(prec):
            want = f32_bits(raw)
            ok = (got.view(np.uint32) == want) | (np.isnan(got) & np.isnan(raw))
            assert np.all(ok), (kind, prec, int((~ok).sum()), np.flatnonzero(~ok)[:5])
        else:
            tc_check(prec, got, raw)


def _rel_2m10(prec, got, raw):
    fin = np.isfinite(raw)
    assert np.array_equal(np.isfinite(got), fin), prec
    rel = np.abs(got[fin] - raw[fin]) / np.maximum(np.abs(raw[fin]), 1e-300)
    assert np.all(rel <= 2.0 ** -10), (prec, rel.max())


# d-4: all-f64, all-f32, all-f16 and the configuration the sweep selects
# (profiles/bench_contract_r1w.json, bench_corr_r1w.json)
def test_2mm_n8192_64_full_rows(torch):
    rng = np.random.default_rng(1)
    rows = _tile_rows(8192, rng, 64)
    run_rows(torch, "2mm", [8192], "random", [[0] * 5, [1] * 5, [2] * 5, [2, 2, 1, 1, 1]], 4, rows,
             np.arange(8192), tc_check=_rel_2m10)


def test_3mm_n8192_tile_grid(torch):
    """3MM's G entries need whole rows of E and columns of F (2 x 67M fmas each): a
    32 x 32 grid with one row per 256-row tile-row and one column per tile-column."""
    rng = np.random.default_rng(2)
    rows = _tile_rows(8192, rng, 32)
    cols = _tile_rows(8192, rng, 32)
    run_rows(torch, "3mm", [8192], "random", [[0] * 7, [1] * 7, [2] * 7, [2, 2, 2, 2, 1, 1, 1]], 6, rows,
             cols, tc_check=_rel_2m10)


def _r6_unit_columns(scale):
    """R6 for a SYRK over columns of unit (CORR: normalised) or bounded norm: by
    Cauchy-Schwarz sum_k |a_k b_k| <= |a| |b| <= scale, so
    |gpu - oracle| <= 2 gamma_N(2^-24) scale + 2 ulp(out)."""
    def chk(prec, got, raw):
        n = 8192
        g = n * 2.0 ** -24 / (1 - n * 2.0 ** -24)
        ulp = np.spacing(np.abs(raw).astype(np.float16 if prec[-1] == 2 else np.float32)).astype(np.float64)
        fin = np.isfinite(raw)
        assert np.array_equal(np.isfinite(got), fin), prec
        err = np.abs(got[fin].astype(np.float64) - raw[fin])
        assert np.all(err <= 2 * g * scale + 2 * ulp[fin]), (prec, err.max())
    return chk


@pytest.mark.parametrize("kind", ["corr", "covar"])
def test_corr_covar_n8192_64_full_rows(torch, kind):
    rng = np.random.default_rng(3)
    rows = _tile_rows(8192, rng, 64)
    m = 4 if kind == "corr" else 3
    so = m - 1
    best = [2, 2, 1, 2] if kind == "corr" else [2, 2, 1]
    cfgs = [[0] * m, [1] * m, [2] * m, best]
    # COVAR: columns of centred U[0,1) data: |col|^2 / (n-1) <= max var-ish; bound the
    # sum by n * (1/2)^2 / (n - 1) (|x - mean| <= 1/2 + tiny for data in [0, 1))
    scale = 1.0 if kind == "corr" else 8192 * 0.25 / 8191 * 1.01
    run_rows(torch, kind, [8192, 8192], "random", cfgs, so, rows, np.arange(8192),
             tc_check=_r6_unit_columns(scale))


@pytest.mark.parametrize("iset", ["default", "random"])
@pytest.mark.parametrize("kind,dims,outs", [("bicg", [16384, 16384], [2, 4]),
                                            ("gesummv", [16384], [3]),
                                            ("atax", [16384, 16384], [2])])
def test_matvec_n16384_every_A_precision(torch, kind, dims, outs, iset):
    """Every precision of A (the 1 GiB object), Table 4 Default and Random inputs,
    256 sampled outputs, bit-exact (mat-vec statements are SIMT, R5)."""
    rng = np.random.default_rng(4)
    n = dims[-1] if kind != "gesummv" else dims[0]
    samples = {k: _vec_samples(n, rng) for k in outs}
    M = 4 if kind == "atax" else 5
    cfgs = []
    for pa in (0, 1, 2):
        c = [pa] + [1] * (M - 1)
        cfgs.append(c)
        if kind == "gesummv":
            cfgs.append([pa, pa] + [1] * (M - 2))
    cfgs.append([2] * M)
    run(torch, kind, dims, iset, cfgs, samples)
