"""C-ABI checks that need no GPU: librap.so builds for sm_100a, loads, exports
every symbol include/rap.h declares, and validates graphs with the same codes
as the oracle (validation runs before any CUDA call)."""
import os
import re
import subprocess

import numpy as np
import pytest

from tests.helpers import node, spec

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def rap():
    from paper_conf_asplos_wangwdz0d24_b200 import _build, rap as r

    _build.build()
    r.load()
    return r


def test_exports_every_declared_symbol(rap):
    hdr = open(os.path.join(ROOT, "include", "rap.h")).read()
    declared = set(re.findall(r"\b(rap_[a-z_]+)\s*\(", hdr))
    declared -= {"rap_plan"}  # struct tag
    assert declared == set(rap.EXPORTS), declared ^ set(rap.EXPORTS)
    from paper_conf_asplos_wangwdz0d24_b200 import _build

    syms = subprocess.run(["nm", "-D", "--defined-only", _build.LIB], capture_output=True, text=True).stdout
    for name in declared:
        assert re.search(rf"\bT {name}\b", syms), name
        assert hasattr(rap.load(), name)


def test_kernel_is_sm100a(rap):
    from paper_conf_asplos_wangwdz0d24_b200 import _build

    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _build.LIB], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_status_strings(rap):
    L = rap.load()
    for code, name in rap.STATUS.items():
        assert L.rap_status_string(code).decode() == ("RAP_ERR_" + name if code else "RAP_OK")


INVALID = {
    "INVALID_GRAPH": [
        spec(1, 1, [node("logit", [("s", 0)], eps=1e-6)], [0]),
        spec(1, 1, [node("firstx", [("n", 1)], x=1), node("firstx", [("n", 0)], x=1)], [0]),
        spec(1, 1, [node("firstx", [("s", 3)], x=1)], [0]),
        spec(1, 1, [node("firstx", [("s", 0)], x=1)], [5]),
        spec(1, 1, [node(42, [("s", 0)])], [0]),
        spec(1, 1, [node("onehot", [("d", 0)], k=4)], [0]),
    ],
    "INVALID_PARAM": [
        spec(1, 0, [node("logit", [("d", 0)], eps=0.5)], [0]),
        spec(1, 0, [node("logit", [("d", 0)], eps=0.0)], [0]),
        spec(1, 0, [node("fillnull", [("d", 0)], f_fill=float("nan"))], [0]),
        spec(1, 0, [node("boxcox", [("d", 0)], **{"lambda": float("inf")})], [0]),
        spec(1, 0, [node("bucketize", [("d", 0)], borders=np.array([1.0, 0.0], dtype=np.float32))], [0]),
        spec(1, 0, [node("bucketize", [("d", 0)], borders=np.array([0.0, np.nan], dtype=np.float32))], [0]),
        spec(0, 1, [node("bucketize", [("s", 0)], borders=np.array([3, 2], dtype=np.int64))], [0]),
        spec(0, 1, [node("sigridhash", [("s", 0)], salt=1, max_value=0)], [0]),
        spec(0, 1, [node("firstx", [("s", 0)], x=-1)], [0]),
        spec(0, 1, [node("clamp", [("s", 0)], lo=5, hi=4)], [0]),
        spec(0, 1, [node("ngram", [("s", 0)], n=9, salt=1, max_value=10)], [0]),
        spec(0, 1, [node("ngram", [("s", 0)] * 9, n=2, salt=1, max_value=10)], [0]),
        spec(0, 1, [node("mapid", [("s", 0)], keys=[1, 1], vals=[2, 3])], [0]),
        spec(0, 1, [node("onehot", [("s", 0)], k=0)], [0]),
        spec(0, 1, [node("onehot", [("s", 0)], k=4097)], [0]),
    ],
}


def test_validation_codes_match_oracle(rap, orc):
    for want, specs in INVALID.items():
        for s in specs:
            assert orc.validate(s)[0] == want, s
            assert rap.validate_only(s) == want, s


def test_output_dims_match_oracle(rap, orc):
    from paper_conf_asplos_wangwdz0d24_b200 import synth

    for name, fn in synth.WORKLOADS.items():
        w = fn(0) if name != "c4" else fn(0, n_features=16)
        st, d, f = orc.validate(w.spec)
        assert st == "OK"
        assert synth.output_dims(w.spec) == (d, f)
