"""Closed-form pins of the quality metric (mean relative error; TOQ
test 'Accuracy < TOQ' fails, Alg. 1 line 10; reading #7)."""
import numpy as np
import pytest

import oracle


def test_identical_output_quality_one(oracle_lib):
    ref = np.linspace(-3, 7, 101)
    r = oracle.quality(ref.copy(), 0, ref)
    assert r["quality"] == 1.0 and r["max_rel"] == 0.0 and r["nonfinite"] == 0


@pytest.mark.parametrize("delta", [1e-3, -0.25, 0.5, 2.0**-11])
def test_uniform_relative_perturbation(oracle_lib, delta):
    ref = np.linspace(1, 9, 333)
    out = ref * (1 + delta)
    r = oracle.quality(out, 0, ref)
    assert r["mean_rel"] == pytest.approx(abs(delta), rel=1e-12)
    assert r["quality"] == pytest.approx(1 - abs(delta), rel=1e-12)


def test_error_capped_at_one_and_overflow(oracle_lib):
    ref = np.ones(10)
    out = ref.copy()
    out[3] = 100.0            # relative error 99 -> capped at 1
    out[5] = np.inf           # overflow -> e = 1, non-finite
    r = oracle.quality(out, 0, ref)
    assert r["quality"] == pytest.approx(1 - 2 / 10, abs=1e-15)
    assert r["nonfinite"] == 1 and r["max_rel"] == np.inf


def test_zero_reference(oracle_lib):
    ref = np.array([0.0, 0.0, 1.0])
    r = oracle.quality(np.array([0.0, -0.0, 1.0]), 0, ref)
    assert r["quality"] == 1.0                       # -0 == 0
    r = oracle.quality(np.array([1e-30, 0.0, 1.0]), 0, ref)
    assert r["quality"] == pytest.approx(2 / 3, abs=1e-15) and r["max_rel"] == np.inf


def test_f16_output_single_overflow(oracle_lib):
    n = 64
    ref = np.full(n, 100.0)
    out = np.full(n, 100.0, dtype=np.float16)
    out[7] = np.inf
    r = oracle.quality(out, 2, ref)
    assert r["quality"] == pytest.approx(1 - 1 / n, abs=1e-15)
    assert r["nonfinite"] == 1


def test_pass_rule_is_q_ge_toq(oracle_lib):
    """P:226 'if Accuracy < TOQ then fail': Q == TOQ passes."""
    objs = oracle.app_objects("gemm", [4])
    ins = [np.ones((4, 4), np.float32)] * 3
    ref = oracle.reference("gemm", [4], ins, scalars=(1.0, 0.0))
    r, _ = oracle.evaluate("gemm", [4], [1, 1, 1], ins, ref, scalars=(1.0, 0.0), toq=1.0)
    assert r["quality"] == 1.0 and r["pass"]
