"""Decision Maker host logic (decision.py, Alg. 1 + Alg. 2) on a fake app: the
wildcard test (Alg. 1 lines 14-32) keeps a measured wildcard configuration only if
it passes AND beats the measured best, and with verify=False accepts an
unverified wildcard on its expected time without a RunApp call."""
import pytest

from paper_conf_cgo_kangcp20_b200 import binding as B
from paper_conf_cgo_kangcp20_b200 import decision as D

N = 1 << 20


def _db(transient_ms=0.1, direct_ms=5.0):
    ents = []
    for dst in (B.F64, B.F32, B.F16):
        for m in D.METHODS:
            ms = transient_ms if m == B.XFER_TRANSIENT else direct_ms
            ents += [{"method": m, "dst": dst, "n": n, "ms": ms * n / N} for n in (N // 4, N)]
    return {"static": {}, "entries": ents}


class FakeApp:
    """M input objects; run_config_host returns a fixed table of (total, transfer, pass)."""
    def __init__(self, m, table):
        self.objects = [{"name": "o%d" % k, "role": 0, "n": N, "rows": 1, "cols": N, "is_output": k == 0}
                        for k in range(m)]
        self.num_objects = m
        self.space = 3 ** m
        self.table = table
        self.calls = []

    def run_config_host(self, prec, host, methods, threads=0, toq=0.9):
        key = (tuple(prec), tuple(methods))
        self.calls.append(key)
        total, transfer, ok = self.table(prec, methods)
        return {"total_ms": total, "transfer_ms": transfer, "quality": 1.0 if ok else 0.0, "pass": ok}


def test_measured_wildcard_must_beat_the_measured_best():
    # one object: f64 10 ms, f32 8 ms, f16 fails -> failed type = f16 = the transient
    # intermediate, so the wildcard (f32 via f16) is measured: 20 ms, slower -> rejected
    def table(prec, meth):
        if meth[0] == B.XFER_TRANSIENT:
            return 20.0, 19.0, True
        return {B.F64: (10.0, 5.0, True), B.F32: (8.0, 5.0, True), B.F16: (4.0, 2.0, False)}[prec[0]]
    app = FakeApp(1, table)
    res = D.decide(app, [None], _db(), toq=0.9, verify=True)
    assert res["prec"] == [B.F32] and res["methods"][0] != B.XFER_TRANSIENT
    assert res["result"]["total_ms"] == 8.0
    assert any(c[1][0] == B.XFER_TRANSIENT for c in app.calls)      # it was measured


def test_unverified_wildcard_accepted_on_expected_time():
    # f16 passes (no failure), so the intermediate is not the failed type: with
    # verify=False the wildcard is taken on its expected time, run once for the report
    def table(prec, meth):
        if meth[0] == B.XFER_TRANSIENT:
            return 3.0, 0.2, True
        return {B.F64: (10.0, 5.0, True), B.F32: (8.0, 5.0, True), B.F16: (9.0, 5.0, True)}[prec[0]]
    app = FakeApp(1, table)
    res = D.decide(app, [None], _db(), toq=0.9, verify=False)
    assert res["methods"][0] == B.XFER_TRANSIENT
    assert sum(1 for c in app.calls if c[1][0] == B.XFER_TRANSIENT) == 1   # only the final report run
    assert res["result"]["total_ms"] == 3.0
