"""Pins for the oracle's applications, codec and quality.

Independent references: numpy float64 textbook linear algebra (matmul, matvec,
np.corrcoef, np.cov), exact integer arithmetic, IEEE error bounds, and closed
forms derived from the paper's definitions.
"""
import itertools

import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import inputs as gen

F64, F32, F16 = 0, 1, 2


# ------------------------------------------------------------------ codec
def test_codec_space_is_3_pow_m_and_bijective(oracle_lib):
    for m in range(1, 8):
        seen = set()
        for cid in range(3 ** m):
            p = oracle.config_decode(m, cid)
            assert oracle.config_encode(p) == cid
            seen.add(tuple(p))
        assert len(seen) == 3 ** m
        assert oracle.config_decode(m, 0) == [F64] * m                    # all-fp64 reference
        assert oracle.config_decode(m, (3 ** m - 1) // 2) == [F32] * m     # original program
        assert oracle.config_decode(m, 3 ** m - 1) == [F16] * m
        with pytest.raises(ValueError):
            oracle.config_decode(m, 3 ** m)


def test_gemm_space_is_27(oracle_lib):
    """(1 + #Conv_Types)^N = (1+2)^3 = 27 for the 3-object example."""
    assert len(oracle.app_objects("gemm", [64])) == 3
    assert 3 ** 3 == 27
    assert (1 + 5 * 2) ** 3 == 1331          # P:127, five methods (Eq. 1 counting)


def test_object_tables(oracle_lib):
    exp = {"gemm": 3, "2mm": 5, "3mm": 7, "atax": 4, "bicg": 5, "gesummv": 5, "corr": 4, "covar": 3}
    for k, n in exp.items():
        objs = oracle.app_objects(k, [8])
        assert len(objs) == n
        assert any(o["is_output"] for o in objs)
    with pytest.raises(ValueError):
        oracle.app_objects("nope", [8])
    with pytest.raises(ValueError):
        oracle.app_objects("gemm", [8, 8])


# ----------------------------------------------------- f64 vs numpy textbook
DIMS = {"gemm": [13, 17, 11], "2mm": [9, 14, 11, 7], "3mm": [6, 9, 8, 10, 7],
        "atax": [37, 45], "bicg": [41, 33], "gesummv": [29], "corr": [40, 23], "covar": [35, 19],
        "mvt": [43], "syrk": [31, 18], "conv2d": [17, 23], "syr2k": [27, 15], "conv3d": [7, 9, 11],
        "fdtd2d": [4, 13, 17]}
CONV2D_C = [0.2, -0.3, 0.4, 0.5, 0.6, 0.7, -0.8, -0.9, 0.10]


def numpy_ref(kind, ins, objs, scalars=None, dims=None):
    A = [None if a is None else a.astype(np.float64).reshape(o["rows"], o["cols"])
         for a, o in zip(ins, objs)]
    if kind == "gemm":
        al, be = scalars or (32412.0, 2123.0)
        return {2: al * (A[0] @ A[1]) + be * A[2]}
    if kind == "2mm":
        C = A[0] @ A[1]
        return {2: C, 4: C @ A[3]}
    if kind == "3mm":
        E = A[0] @ A[1]
        F = A[2] @ A[3]
        return {4: E, 5: F, 6: E @ F}
    if kind == "atax":
        tmp = A[0] @ A[1][0]
        return {3: tmp[None, :], 2: (A[0].T @ tmp)[None, :]}
    if kind == "bicg":
        return {2: (A[0].T @ A[1][0])[None, :], 4: (A[0] @ A[3][0])[None, :]}
    if kind == "gesummv":
        al, be = scalars or (43532.0, 12313.0)
        tmp = A[0] @ A[2][0]
        y = A[1] @ A[2][0]
        return {4: tmp[None, :], 3: (al * tmp + be * y)[None, :]}
    if kind == "corr":
        c = np.corrcoef(A[0], rowvar=False)
        return {3: c}
    if kind == "covar":
        return {2: np.cov(A[0], rowvar=False)}
    if kind == "mvt":
        return {1: (A[1][0] + A[0] @ A[3][0])[None, :], 2: (A[2][0] + A[0].T @ A[4][0])[None, :]}
    if kind == "syrk":      # BLAS 'T' form; the result's lower triangle mirrors the upper
        al, be = scalars or (32412.0, 2123.0)
        cu = np.triu(A[1])
        c = cu + np.triu(cu, 1).T
        return {1: al * (A[0].T @ A[0]) + be * c}
    if kind == "conv2d":
        a = A[0]
        b = np.zeros_like(a)
        di = [-1, 0, 1] * 3
        dj = [-1] * 3 + [0] * 3 + [1] * 3
        ni, nj = a.shape
        for c, x, y in zip(CONV2D_C, di, dj):
            b[1:-1, 1:-1] += c * a[1 + x:ni - 1 + x, 1 + y:nj - 1 + y]
        return {1: b}
    if kind == "syr2k":
        al, be = scalars or (32412.0, 2123.0)
        return {2: al * (A[0].T @ A[1] + A[1].T @ A[0]) + be * A[2]}
    if kind == "conv3d":
        ni, nj, nk = dims
        a = A[0].reshape(ni, nj, nk)
        b = np.zeros_like(a)
        for p, g in enumerate((0.25, 0.5, 0.25)):
            for q, c in enumerate(CONV2D_C):
                di, dj, dk = p - 1, q % 3 - 1, q // 3 - 1
                b[1:-1, 1:-1, 1:-1] += g * c * a[1 + di:ni - 1 + di, 1 + dj:nj - 1 + dj, 1 + dk:nk - 1 + dk]
        return {1: b.reshape(ni, nj * nk)}
    if kind == "fdtd2d":
        tmax = objs[0]["cols"]
        fict, ex, ey, hz = A[0][0].copy(), A[1].copy(), A[2].copy(), A[3].copy()
        for t in range(tmax):
            ey[0, :] = fict[t]
            ey[1:, :] = ey[1:, :] - 0.5 * (hz[1:, :] - hz[:-1, :])
            ex[:, 1:] = ex[:, 1:] - 0.5 * (hz[:, 1:] - hz[:, :-1])
            hz[:-1, :-1] = hz[:-1, :-1] - 0.7 * (ex[:-1, 1:] - ex[:-1, :-1] + ey[1:, :-1] - ey[:-1, :-1])
        return {1: ex, 2: ey, 3: hz}
    raise KeyError(kind)


@pytest.mark.parametrize("kind", sorted(DIMS))
@pytest.mark.parametrize("iset", ["default", "random"])
def test_f64_config_matches_numpy(oracle_lib, kind, iset):
    if kind in ("corr", "covar") and iset == "default":
        pytest.skip("default inputs are rank-1 (degenerate correlations); random set used")
    dims = DIMS[kind]
    objs = oracle.app_objects(kind, dims)
    ins = gen.make_inputs(kind, objs, iset, seed=3)
    fin = oracle.reference(kind, dims, ins)
    for m, want in numpy_ref(kind, ins, objs, dims=dims).items():
        got = fin[m]
        assert got.dtype == np.float64
        np.testing.assert_allclose(got, want, rtol=1e-12, atol=1e-12 * np.abs(want).max())


def test_corr_diagonal_is_one_and_symmetric(oracle_lib):
    dims = [50, 12]
    objs = oracle.app_objects("corr", dims)
    ins = gen.make_inputs("corr", objs, "random")
    for prec in ([0, 0, 0, 0], [1, 1, 1, 1], [2, 1, 1, 2]):
        s = oracle.run_config("corr", dims, prec, ins)[3].astype(np.float64)
        assert np.array_equal(s, s.T)
        assert np.all(np.diag(s) == 1.0)


def test_corr_eps_guard(oracle_lib):
    """A constant column has stddev 0 <= eps -> replaced by 1 (PolyBench-shaped)."""
    dims = [20, 5]
    objs = oracle.app_objects("corr", dims)
    ins = gen.make_inputs("corr", objs, "random")
    ins[0] = ins[0].copy()
    ins[0][:, 2] = 7.0
    fin = oracle.run_config("corr", dims, [0, 0, 0, 0], ins)
    assert fin[2][0, 2] == 1.0
    assert np.all(fin[3][2, [0, 1, 3, 4]] == 0.0)


# -------------------------------------------- exact-integer invariants (R3/R5)
def _exact_ints(kind, dims, objs, rng, lo=0, hi=8):
    ins = []
    for o in objs:
        ins.append(rng.integers(lo, hi, size=(o["rows"], o["cols"])).astype(np.float32)
                   if o["role"] in (0, 2) else None)
    return ins


def _fits(v, p):
    lim = {F64: 2.0 ** 53, F32: 2.0 ** 24, F16: 2048.0}[p]
    return np.all(np.abs(v) <= lim)


@pytest.mark.parametrize("kind", ["gemm", "2mm", "3mm", "atax", "bicg", "gesummv", "mvt", "syrk",
                                  "syr2k"])
def test_exact_integer_results_every_config(oracle_lib, kind):
    """With small non-negative integer inputs every partial sum is an integer
    bounded by the final value, so every configuration whose objects can hold
    those integers exactly must reproduce exact integer arithmetic -- whatever
    the reduction order (pins indices/transposes/dropped terms of R3 and R5,
    including ragged lanes and chunk tails)."""
    rng = np.random.default_rng(7)
    dims = {"atax": [300, 77], "bicg": [270, 93], "gesummv": [75]}.get(kind, DIMS[kind])
    objs = oracle.app_objects(kind, dims)
    ins = _exact_ints(kind, dims, objs, rng)
    sc = (2.0, 3.0) if kind in ("gemm", "gesummv", "syrk", "syr2k") else None
    if kind == "syrk":        # C must be symmetric for the textbook form to apply
        ins[1] = np.triu(ins[1]) + np.triu(ins[1], 1).T
    exact = {m: np.rint(v) for m, v in numpy_ref(kind, ins, objs, sc, dims).items()}
    n_checked = 0
    for prec in itertools.product([F64, F32, F16], repeat=len(objs)):
        if not all(_fits(v, prec[m]) for m, v in exact.items()):
            continue
        fin = oracle.run_config(kind, dims, list(prec), ins, sc)
        for m, v in exact.items():
            assert np.array_equal(fin[m].astype(np.float64).reshape(v.shape), v), (prec, m)
        n_checked += 1
    assert n_checked >= 3 ** len(objs) // 4


def test_colsum_chunk_tail_exact(oracle_lib):
    """ATAX with NX spanning several 256-row chunks plus a ragged tail."""
    dims = [2 * oracle.COLSUM_CHUNK + 17, 40]
    objs = oracle.app_objects("atax", dims)
    rng = np.random.default_rng(11)
    ins = _exact_ints("atax", dims, objs, rng, 0, 4)
    fin = oracle.run_config("atax", dims, [F32] * 4, ins)
    ref = numpy_ref("atax", ins, objs)
    assert np.array_equal(fin[2].astype(np.float64), ref[2])


def test_rowdot_slab_and_tile_tails_exact(oracle_lib):
    """Rows spanning several 8-slab tiles with a ragged last slab, every precision
    of A: exact integer results (no dropped or duplicated slab/tile)."""
    dims = [9, 8 * 32 * 8 * 2 + 3 * 32 + 5]     # > 2 f16 tiles, > 4 f32 tiles, > 8 f64 tiles
    objs = oracle.app_objects("atax", dims)
    rng = np.random.default_rng(13)
    ins = _exact_ints("atax", dims, objs, rng, 0, 4)
    ref = numpy_ref("atax", ins, objs)
    for pa in (F64, F32, F16):
        fin = oracle.run_config("atax", dims, [pa, F32, F64, F64], ins)
        assert np.array_equal(fin[3].astype(np.float64), ref[3]), pa
        assert np.array_equal(fin[2].astype(np.float64), ref[2]), pa


# ---------------------------------------------------------- error bounds
@pytest.mark.parametrize("kind", ["gemm", "atax", "bicg", "gesummv", "2mm"])
def test_all_f32_within_gamma_bound(oracle_lib, kind):
    """Positive inputs: |fl(sum) - sum| <= gamma_K * sum (+ output rounding)."""
    dims = DIMS[kind]
    objs = oracle.app_objects(kind, dims)
    ins = gen.make_inputs(kind, objs, "random", seed=5)
    ref = oracle.reference(kind, dims, ins)
    fin = oracle.run_config(kind, dims, [F32] * len(objs), ins)
    K = max(max(o["rows"], o["cols"]) for o in objs)
    u = 2.0 ** -24
    depth = 2 if kind == "2mm" else 1
    bound = (depth * (K + 4)) * u / (1 - depth * (K + 4) * u)
    for m, o in enumerate(objs):
        if o["is_output"]:
            r = ref[m]
            rel = np.abs(fin[m].astype(np.float64) - r) / np.abs(r)
            assert np.all(rel <= bound), (m, rel.max(), bound)


# ------------------------------------------------------- GEMM-64 (config 1)
def test_gemm64_default_overflow_pin(oracle_lib):
    """BASELINE config 1.  Default inputs (Table 4 GEMM range 0-513) with
    alpha=32412: alpha*(A.B)_ij >= 32412*513^2*85344/63^4 ~ 4.6e7 > 65504 for all
    i,j >= 1, so every config with C in fp16 overflows on the 63*63 interior
    (P:160 'TOQ failure due to the limited range'): Q = 1 - 3969/4096 exactly, fail.
    Every other config rounds inputs to at worst fp16 (relative 2^-11 each):
    Q >= 1 - 2^-9 > TOQ 0.9."""
    objs = oracle.app_objects("gemm", [64])
    ins = gen.make_inputs("gemm", objs, "default")
    ref, res = oracle.sweep("gemm", [64], range(27), ins, toq=0.9)
    n_pass = 0
    for r in res:
        prec = oracle.config_decode(3, r["config_id"])
        if prec[2] == F16:
            assert r["nonfinite"] == 63 * 63
            assert r["quality"] == pytest.approx(1 - 3969 / 4096, abs=1e-15)
            assert not r["pass"] and r["max_rel"] == np.inf
        else:
            assert r["nonfinite"] == 0 and r["pass"]
            assert r["quality"] >= 1 - 2.0 ** -9
            n_pass += 1
    assert n_pass == 18


def test_gemm64_random_all_pass(oracle_lib):
    objs = oracle.app_objects("gemm", [64])
    ins = gen.make_inputs("gemm", objs, "random")
    _, res = oracle.sweep("gemm", [64], range(27), ins, scalars=(1.5, 1.2), toq=0.9)
    assert all(r["pass"] for r in res)


def test_all_f64_config_is_the_reference(oracle_lib):
    """North star invariant: the all-high-precision configuration reproduces the
    fp64 reference exactly (raw outputs)."""
    for kind in DIMS:
        dims = DIMS[kind]
        objs = oracle.app_objects(kind, dims)
        ins = gen.make_inputs(kind, objs, "random")
        a = oracle.reference(kind, dims, ins)
        b = oracle.run_config(kind, dims, [F64] * len(objs), ins)
        for x, y in zip(a, b):
            assert np.array_equal(x, y)


def test_all_f32_config_is_plain_fp32_program_for_exact_inputs(oracle_lib):
    """Id (3^M-1)/2 is the original program: with orig == f32 no conversion is
    applied, so the delivered outputs are the raw f32 outputs."""
    dims = [16]
    objs = oracle.app_objects("gemm", dims)
    ins = gen.make_inputs("gemm", objs, "random")
    ref = oracle.reference("gemm", dims, ins)
    prec = oracle.config_decode(3, 13)
    assert prec == [F32] * 3
    r, delivered = oracle.evaluate("gemm", dims, prec, ins, ref)
    raw = oracle.run_config("gemm", dims, prec, ins)
    assert np.array_equal(delivered[2], raw[2])
