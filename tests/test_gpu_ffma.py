"""f32 contractions on FFMA2 (gemm_ffma.cu): fma.rn.f32x2 must be two independent
IEEE fma.rn per lane -- reading R3's chain bit for bit -- including subnormal
operands, subnormal products and partial sums, overflow to inf and NaN.  The
inputs mix exponents over [-80, 20] (products down to 2^-160: below the f32
subnormal range, so gradual underflow is exercised in every chain), exact zeros,
near-cancelling pairs, and a few inf / NaN; shapes are ragged against the 64 x 128
tile and the 16-deep k tile.  Every configuration whose statements compute in f32
(no f64 object) is compared with the oracle bit for bit."""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B

from test_gpu_apps import check_config, same_bits

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def underflowing(n, seed, special=False):
    rng = np.random.default_rng(seed)
    v = (rng.uniform(0.5, 1.0, n) * np.exp2(rng.integers(-80, 21, n).astype(np.float64))).astype(np.float32)
    v *= np.where(rng.integers(0, 2, n) == 1, -1, 1).astype(np.float32)
    v[rng.integers(0, 9, n) == 0] = 0
    sub = rng.integers(0, 13, n) == 0                     # f32 subnormal operands
    v[sub] = (rng.uniform(-1, 1, int(sub.sum())) * 2.0 ** -127).astype(np.float32)
    pair = np.flatnonzero(rng.integers(0, 7, n) == 0)
    pair = pair[pair > 0]
    v[pair] = -v[pair - 1] * np.float32(1 + 2 ** -20)
    if special:
        idx = rng.choice(n, size=3, replace=False)
        v[idx] = [np.inf, -np.inf, np.nan]
    return v


@pytest.mark.parametrize("kind,dims,sc,special", [
    ("gemm", [257, 131, 203], (1.5, 1.2), False),
    ("gemm", [70, 300, 45], None, True),
    ("syrk", [203, 141], (1.5, 1.2), False),
    ("2mm", [130, 70, 91, 45], None, False),
    ("syr2k", [97, 150], None, False),
])
def test_f32_statements_bit_exact_underflow(torch, kind, dims, sc, special):
    app = B.App(kind, dims, sc)
    app.set_flags(B.FLAG_NO_TENSOR_CORES)
    ins = []
    for m, o in enumerate(app.objects):
        ins.append(underflowing(int(o["n"]), 300 + m, special and m == 0) if o["role"] in (0, 2) else None)
    app.bind([torch.from_numpy(a).cuda() if a is not None else None for a in ins])
    refs = app.reference()
    oref = oracle.reference(kind, dims, ins, sc)
    for m, o in enumerate(app.objects):
        if o["is_output"]:
            assert same_bits(refs[m].cpu().numpy(), oref[m]), "fp64 reference differs (obj %d)" % m
    n_checked = 0
    for cid in range(app.space):
        prec = app.decode(cid)
        if 0 in prec:
            continue          # f64 statements: test_gpu_f64.py
        check_config(torch, app, kind, dims, ins, oref, prec, sc)
        n_checked += 1
    assert n_checked == 2 ** app.num_objects
