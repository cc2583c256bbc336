"""C-ABI library loads and exports every symbol include/prescaler.h declares;
host-only logic (object tables, codec, validation) runs without a GPU."""
import ctypes
import os
import re

import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import binding as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
APPS = {"gemm": [13, 17, 11], "2mm": [9, 14, 11, 7], "3mm": [6, 9, 8, 10, 7],
        "atax": [37, 45], "bicg": [41, 33], "gesummv": [29], "corr": [40, 23], "covar": [35, 19],
        "mvt": [43], "syrk": [31, 18], "conv2d": [17, 23],
        "syr2k": [27, 15], "conv3d": [7, 9, 11], "fdtd2d": [4, 13, 17]}


@pytest.fixture(scope="module")
def lib():
    from paper_conf_cgo_kangcp20_b200 import build
    build.build()
    return B.lib()


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "prescaler.h")).read()
    return sorted(set(re.findall(r"PS_API[^;(]*?\b(ps_\w+)\s*\(", txt)))


def test_header_symbols_match_binding():
    assert header_symbols() == sorted(B.SYMBOLS)


def test_library_exports_every_header_symbol(lib):
    for name in header_symbols():
        assert hasattr(lib, name), name
    assert "sm_100a" in B.ps_version()


def test_status_strings(lib):
    assert B.ps_status_string(0) == "ok"
    assert "workspace" in B.ps_status_string(4)


def test_result_struct_is_64_bytes():
    assert ctypes.sizeof(B.PsResult) == 64


@pytest.mark.parametrize("kind", sorted(APPS))
def test_object_tables_agree_with_oracle(lib, kind):
    """Host logic of the CUDA library vs the oracle's independently written tables."""
    app = B.App(kind, APPS[kind])
    ora = oracle.app_objects(kind, APPS[kind])
    assert app.num_objects == len(ora)
    for a, o in zip(app.objects, ora):
        assert (a["name"], a["role"], a["is_output"], a["rows"], a["cols"]) == \
               (o["name"], o["role"], o["is_output"], o["rows"], o["cols"])
        assert a["orig"] == B.F32 and a["n"] == a["rows"] * a["cols"]
    assert app.workspace_bytes >= sum(o["n"] * 8 for o in app.objects)


@pytest.mark.parametrize("kind", sorted(APPS))
def test_codec_matches_oracle(lib, kind):
    app = B.App(kind, APPS[kind])
    m = app.num_objects
    for cid in range(0, 3 ** m, max(1, 3 ** m // 200)):
        p = app.decode(cid)
        assert p == oracle.config_decode(m, cid)
        assert app.encode(p) == cid
    with pytest.raises(B.PsError):
        app.decode(3 ** m)
    with pytest.raises(B.PsError):
        app.encode([3] * m)


def test_validation(lib):
    with pytest.raises(B.PsError):
        B.App("nope", [4])
    with pytest.raises(B.PsError):
        B.App("gemm", [4, 4])
    with pytest.raises(B.PsError):
        B.App("gemm", [0])
    with pytest.raises(B.PsError):       # bad dtype
        B.ps_convert(0, 5, 0, 1, 4, stream=0)
    with pytest.raises(B.PsError):       # overlap
        B.ps_convert(4096, 1, 4100, 2, 16, stream=0)
    B.ps_convert(0, 1, 0, 2, 0, stream=0)   # n == 0: no-op, no GPU needed
    app = B.App("gemm", [8])
    with pytest.raises(B.PsError):       # not bound
        app.run_config([1, 1, 1], stream=0)
    with pytest.raises(B.PsError):
        app.sweep([0], stream=0)


def test_missing_library_fails_loudly(monkeypatch, tmp_path):
    monkeypatch.setattr(B, "LIB_PATH", str(tmp_path / "absent.so"))
    monkeypatch.setattr(B, "_lib", None)
    with pytest.raises(B.PsError):
        B.lib()
