"""ps_search's trial sequence replayed against the paper's Alg. 1 with the ORACLE's
TOQ decisions.

The native search (prescaler.h (6)) logs every RunApp call (Alg. 1 line 8): the
configuration, its measured time and its pass flag.  Times are measurements, so
they are taken from the log; every pass/fail decision comes from the oracle
(`oracle.sweep`, "Accuracy < TOQ").  The replay below is written from the
paper, not from app.cu:
  * pre-full-precision scaling (Sec. 4.4.1): the uniform configurations in
    descending precision, start from the fastest passing one (all-f64 if none);
  * objects in descending order of data volume (the sum of the execution
    times of the events related to the object; the device-only stand-in is
    elements x statements touching the object -- TOUCH below, read off each app's
    statements);
  * per object (Alg. 1 lines 2-13): targets in descending precision,
    skipping the current type (line 3), stop at the first TOQ failure (line 10),
    keep the fastest passing configuration (line 12), ties to the lower id.
The replay must request exactly the logged configurations in the logged order
and finish on the same choice, and the GPU's pass flags must equal the oracle's.
"""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import inputs as gen

pytestmark = pytest.mark.gpu

# statements reading or writing each object (PolyBench statement lists)
TOUCH = {
    "gemm": [1, 1, 1],                 # C <- alpha A B + beta C
    "atax": [2, 1, 1, 2],              # tmp = A x; y = A^T tmp   (A, x, y, tmp)
    "bicg": [2, 1, 1, 1, 1],           # s = A^T r; q = A p       (A, r, s, p, q)
    "gesummv": [1, 1, 2, 2, 2],        # tmp = A x; y = B x; y = a tmp + b y
    "mvt": [2, 1, 1, 1, 1],            # x1 += A y1; x2 += A^T y2
}


def replay(app, toq, log_ms, oracle_pass):
    m, radix = app.num_objects, app.radix
    enc = lambda p: sum(int(t) * radix ** k for k, t in enumerate(p))
    seq, seen = [], {}

    def run(p):
        cid = enc(p)
        if cid not in seen:
            assert cid in log_ms, "replay asks for config %d, which the native search never ran" % cid
            seen[cid] = (log_ms[cid], oracle_pass[cid])
            seq.append(cid)
        return seen[cid]

    def better(a, ai, b, bi):
        return a[0] < b[0] or (a[0] == b[0] and ai < bi)

    cur, tcur = None, None
    for t in range(radix):                                   # PFP, descending precision
        p = [t] * m
        r = run(p)
        if r[1] and (cur is None or better(r, enc(p), tcur, enc(cur))):
            cur, tcur = p, r
    if cur is None:
        cur = [0] * m
        tcur = run(cur)
    vol = [app.objects[k]["n"] * TOUCH[app.kind][k] for k in range(m)]
    order = sorted(range(m), key=lambda k: (-vol[k], k))
    for k in order:                                          # Alg. 1 per object
        best, tbest = list(cur), tcur
        for t in range(radix):
            if t == cur[k]:
                continue
            p = list(cur)
            p[k] = t
            r = run(p)
            if not r[1]:
                break
            if better(r, enc(p), tbest, enc(best)):
                best, tbest = p, r
        cur, tcur = best, tbest
    return seq, enc(cur)


@pytest.fixture(scope="module")
def torch():
    import torch as t
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    B.lib()
    return t


@pytest.mark.parametrize("kind,dims,iset,toq", [
    ("gemm", [64], "default", 0.9), ("gemm", [96], "random", 0.99),
    ("atax", [512, 768], "default", 0.9), ("bicg", [640, 512], "random", 0.9),
    ("gesummv", [700], "image", 0.9), ("mvt", [600], "random", 0.999),
])
def test_search_trials_replay_alg1(torch, kind, dims, iset, toq):
    app = B.App(kind, dims)
    ins = gen.make_inputs(kind, app.objects, iset)
    app.bind([torch.from_numpy(a.reshape(-1)).cuda() if a is not None else None for a in ins])
    app.reference()
    res = app.search(toq, repeats=1)
    assert res["trials"] <= 64
    oref = oracle.reference(kind, dims, ins)
    _, ores = oracle.sweep(kind, dims, res["trial_ids"], ins, ref=oref, toq=toq)
    opass = {r["config_id"]: bool(r["pass"]) for r in ores}
    # the GPU's TOQ decisions are the oracle's
    assert res["trial_pass"] == [opass[c] for c in res["trial_ids"]]
    log_ms = dict(zip(res["trial_ids"], res["trial_ms"]))
    seq, choice = replay(app, toq, log_ms, opass)
    assert seq == res["trial_ids"]
    assert choice == res["config_id"]
    assert res["pass"] == opass[choice] or choice == 0
