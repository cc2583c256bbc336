"""The oracle's sampled evaluation (used for parity at the BASELINE sizes) equals
its full run bit for bit: same helpers, same orders, only fewer elements."""
import itertools

import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import inputs as gen

CASES = {"gemm": [37, 29, 41], "2mm": [19, 23, 17, 21], "3mm": [11, 13, 9, 15, 10],
         "atax": [300, 77], "bicg": [270, 93], "gesummv": [75], "corr": [60, 17], "covar": [55, 13],
         "mvt": [301], "syrk": [23, 14], "conv2d": [15, 21], "syr2k": [21, 13],
         "conv3d": [6, 7, 9], "fdtd2d": [3, 11, 13]}


@pytest.mark.parametrize("kind", sorted(CASES))
def test_sample_equals_full_run(oracle_lib, kind):
    dims = CASES[kind]
    objs = oracle.app_objects(kind, dims)
    ins = gen.make_inputs(kind, objs, "random", seed=1)
    rng = np.random.default_rng(2)
    m = len(objs)
    ids = sorted(set([0, (3 ** m - 1) // 2, 3 ** m - 1] + list(rng.integers(0, 3 ** m, 6))))
    for cid in ids:
        prec = oracle.config_decode(m, int(cid))
        full = oracle.run_config(kind, dims, prec, ins)
        for k, o in enumerate(objs):
            if not o["is_output"]:
                continue
            rr, cc = np.meshgrid(np.arange(o["rows"]), np.arange(o["cols"]), indexing="ij")
            rr, cc = rr.reshape(-1), cc.reshape(-1)
            pick = rng.choice(rr.size, size=min(rr.size, 40), replace=False)
            pick.sort()
            vals = oracle.sample(kind, dims, prec, ins, k, rr[pick], cc[pick])
            want = full[k].astype(np.float64).reshape(-1)[pick]
            same = (vals.view(np.uint64) == want.view(np.uint64)) | (np.isnan(vals) & np.isnan(want))
            assert np.all(same), (kind, prec, k)


def test_sample_rejects_bad_entries(oracle_lib):
    objs = oracle.app_objects("gemm", [8])
    ins = gen.make_inputs("gemm", objs, "random")
    with pytest.raises(ValueError):
        oracle.sample("gemm", [8], [1, 1, 1], ins, 2, [8], [0])
    with pytest.raises(ValueError):
        oracle.sample("gemm", [8], [1, 1, 1], ins, 0, [0], [0])   # not an output
