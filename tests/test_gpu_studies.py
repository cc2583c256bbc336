"""Fig. 6 / Fig. 12 study drivers (studies.py) on the CUDA path, checked against the
oracle: the all-fp16 quality of every app and input set (Fig. 6) equals the
oracle's (bit-exact on the SIMT apps; tcgen05 contractions within 1e-3, R6),
and the Decision Maker's choice (Fig. 12) passes its TOQ per the oracle."""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

pytestmark = pytest.mark.gpu

TINY = {"gemm": [40], "atax": [300, 70], "bicg": [260, 90], "gesummv": [130], "corr": [70, 33],
        "covar": [65, 30], "mvt": [300], "syrk": [70, 40], "conv2d": [40, 70], "syr2k": [66, 40],
        "conv3d": [10, 20, 70], "fdtd2d": [4, 40, 70], "2mm": [40, 50, 30, 20],
        "3mm": [20, 30, 40, 25, 35]}
TC_APPS = {"gemm", "2mm", "3mm", "corr", "covar", "syrk", "syr2k"}


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


def test_fig6_matches_oracle(torch):
    from paper_conf_cgo_kangcp20_b200 import studies
    res = studies.fig6(torch, TINY)
    for kind, dims in TINY.items():
        objs = oracle.app_objects(kind, dims)
        for iset in studies.INPUT_SETS:
            ins = gen.make_inputs(kind, objs, iset)
            ro, _ = oracle.evaluate(kind, dims, [2] * len(objs), ins, oracle.reference(kind, dims, ins),
                                    toq=0.9)
            got = res[kind][iset]
            if kind in TC_APPS:
                assert abs(got["quality"] - ro["quality"]) <= 1e-3, (kind, iset)
            else:
                assert got["quality"] == round(ro["quality"], 6), (kind, iset)
                assert got["nonfinite"] == ro["nonfinite"]


def test_fig12_choice_passes_toq(torch):
    from paper_conf_cgo_kangcp20_b200 import decision as D
    from paper_conf_cgo_kangcp20_b200 import studies
    db = D.inspect(sizes=(1 << 16, 1 << 20), reps=1)
    sizes = {k: TINY[k] for k in ("atax", "conv2d", "fdtd2d")}
    res = studies.fig12(torch, db, sizes, cases=[("default", 0.9), ("random", 0.99)], reps=1)
    summ = studies.summarize(res)
    assert set(summ) == {"default@0.90", "random@0.99"}
    for kind, row in res.items():
        objs = oracle.app_objects(kind, TINY[kind])
        for case, r in row.items():
            iset, toq = case.split("@")
            ins = gen.make_inputs(kind, objs, iset)
            ro, _ = oracle.evaluate(kind, TINY[kind], r["chosen"], ins,
                                    oracle.reference(kind, TINY[kind], ins), toq=float(toq))
            assert ro["pass"], (kind, case, r["chosen"])
            assert 0.0 <= r["half_fraction"] <= 1.0 and r["trials"] <= 3 * len(objs) + 3 + 2 * len(objs)
            dev = r["device_only_exhaustive"]
            assert dev is not None and dev["passing"] >= 1


def test_bf16_gain_structure(torch):
    from paper_conf_cgo_kangcp20_b200 import studies
    res = studies.bf16_gain(torch, {"gemm": [64], "atax": [300, 70]}, input_sets=("default",))
    for kind, row in res.items():
        r = row["default"]
        # the 4^M space contains the 3^M one: at least as many passing configs, and a
        # best that is no slower than the paper-space best (up to timing noise)
        assert r["bf16_4^M"]["passing"] >= r["paper_3^M"]["passing"]
        assert r["bf16_4^M"]["space"] == 4 ** len(r["bf16_4^M"]["best_prec"])
