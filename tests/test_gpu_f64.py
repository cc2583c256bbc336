"""f64 contractions: the DMMA kernel (gemm_dmma.cu, the default) and the DFMA
kernel (gemm_simt.cuh, PS_F64_DFMA=1) are both bit-exact (and so are both f32 kernels) with reading R3's fma
chain.  The DMMA kernel relies on mma.sync .f64 computing fma(a3,b3, ... fma(a0,b0,c))
(measured: profiles/dmma_probe_r1.txt); these inputs are built so that any other
summation order or a fused dot product would change results: wide exponent
ranges, cancellation, exact zeros, K not a multiple of 4 or 16, ragged M / N."""
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B

from test_gpu_apps import check_config, same_bits

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def adversarial(n, seed):
    """float32 values with exponents over [-20, 20], random signs, 1 in 9 exactly zero,
    1 in 7 a near-cancelling partner of the previous value."""
    rng = np.random.default_rng(seed)
    v = (rng.uniform(0.5, 1.0, n) * np.exp2(rng.integers(-20, 21, n))).astype(np.float32)
    v *= np.where(rng.integers(0, 2, n) == 1, -1, 1).astype(np.float32)
    v[rng.integers(0, 9, n) == 0] = 0
    pair = np.flatnonzero(rng.integers(0, 7, n) == 0)
    pair = pair[pair > 0]
    v[pair] = -v[pair - 1] * np.float32(1 + 2 ** -20)
    return v


@pytest.mark.parametrize("kind,dims,sc", [("gemm", [257, 131, 203], (1.5, 1.2)),
                                          ("gemm", [64, 200, 37], None),
                                          ("syrk", [203, 141], (1.5, 1.2)),
                                          ("2mm", [130, 70, 91, 45], None)])
def test_f64_statements_bit_exact_adversarial(torch, kind, dims, sc):
    app = B.App(kind, dims, sc)
    app.set_flags(B.FLAG_NO_TENSOR_CORES)
    ins = []
    for m, o in enumerate(app.objects):
        ins.append(adversarial(int(o["n"]), 100 + m) if o["role"] in (0, 2) else None)
    app.bind([torch.from_numpy(a).cuda() if a is not None else None for a in ins])
    refs = app.reference()
    oref = oracle.reference(kind, dims, ins, sc)
    for m, o in enumerate(app.objects):
        if o["is_output"]:
            assert same_bits(refs[m].cpu().numpy(), oref[m]), "fp64 reference differs (obj %d)" % m
    # every configuration whose contraction runs in f64, plus all-f32 for contrast
    M = app.num_objects
    for cid in range(app.space):
        prec = app.decode(cid)
        if 0 in prec or cid == (3 ** M - 1) // 2:
            check_config(torch, app, kind, dims, ins, oref, prec, sc)


def test_dmma_self_check_selects_dmma_on_b200():
    """ps_f64_uses_dmma: the per-device self-check (adversarial 128x128x64 product,
    DMMA vs DFMA bit for bit) passes on B200, so f64 statements run on DMMA."""
    from paper_conf_cgo_kangcp20_b200 import binding as B
    assert B.lib().ps_f64_uses_dmma() == 1


@pytest.mark.parametrize("switch", ["PS_F64_DFMA"])
def test_fallback_kernel_bit_exact(switch):
    """The DFMA f64 kernel (the self-check fallback, forced by PS_F64_DFMA=1) stays
    R3-exact: the contraction apps' exhaustive SIMT parity cases in a child process."""
    env = dict(os.environ, **{switch: "1"})
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider", "-m", "gpu",
                        os.path.join(ROOT, "tests", "test_gpu_apps.py"),
                        "-k", "gemm or 2mm or 3mm or corr or covar or syrk or syr2k"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=1800)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
