"""ctypes wrapper around the C oracle (oracle/rap_oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, ``__graft_entry__.smoke()`` and
bench.py's ``cpu_baseline`` / ``--impl reference`` legs may import this module.
The product package (paper_conf_asplos_wangwdz0d24_b200) never imports it.

The graph-spec format (a plain dict) is an input description
shared with the product binding the same way the seeded input generator is;
this wrapper turns it into the oracle's own C structs.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "rap_oracle.c")
LIB = os.path.join(HERE, "liborc.so")

OPS = {"fillnull": 0, "logit": 1, "boxcox": 2, "onehot": 3, "sigridhash": 4,
       "bucketize": 5, "firstx": 6, "clamp": 7, "ngram": 8, "mapid": 9}
STATUS = {0: "OK", 1: "INVALID_ARGUMENT", 2: "INVALID_GRAPH", 3: "INVALID_PARAM",
          4: "CAPACITY", 5: "UNSUPPORTED", 7: "OUT_OF_MEMORY"}
IN_KIND = {"n": 0, "d": 1, "s": 2}
MAX_IN = 8


class OrcNode(C.Structure):
    _fields_ = [("op", C.c_int32), ("n_in", C.c_int32),
                ("in_kind", C.c_int32 * MAX_IN), ("in_idx", C.c_int32 * MAX_IN),
                ("f_fill", C.c_float), ("eps", C.c_float), ("lam", C.c_float),
                ("i_fill", C.c_int64), ("lo", C.c_int64), ("hi", C.c_int64), ("x", C.c_int64),
                ("max_value", C.c_int64), ("map_default", C.c_int64), ("salt", C.c_uint64),
                ("n", C.c_int32), ("k_width", C.c_int32), ("n_borders", C.c_int32),
                ("f_borders", C.c_void_p), ("i_borders", C.c_void_p),
                ("map_size", C.c_int64), ("map_keys", C.c_void_p), ("map_vals", C.c_void_p)]


class OrcGraph(C.Structure):
    _fields_ = [("n_dense", C.c_int32), ("n_sparse", C.c_int32), ("n_nodes", C.c_int32),
                ("nodes", C.POINTER(OrcNode)), ("n_outputs", C.c_int32), ("outputs", C.POINTER(C.c_int32))]


class OrcBatch(C.Structure):
    _fields_ = [("n_rows", C.c_int64), ("dense", C.POINTER(C.c_void_p)), ("dense_valid", C.POINTER(C.c_void_p)),
                ("sp_off", C.POINTER(C.c_void_p)), ("sp_val", C.POINTER(C.c_void_p)),
                ("sp_valid", C.POINTER(C.c_void_p))]


class OrcResult(C.Structure):
    _fields_ = [("n_rows", C.c_int64), ("d_out", C.c_int64), ("f_out", C.c_int64), ("n_values", C.c_int64),
                ("dense", C.POINTER(C.c_float)), ("lengths", C.POINTER(C.c_int32)),
                ("offsets", C.POINTER(C.c_int64)), ("values", C.POINTER(C.c_int64))]


_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain C11, no fast-math, no FP contraction)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(
            os.path.getmtime(SRC), os.path.getmtime(os.path.join(HERE, "rap_oracle.h"))):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-std=c11", "-O1", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-o", tmp, SRC, "-lm"])
        os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(LIB)
            L.orc_H.restype = C.c_uint64
            L.orc_H.argtypes = [C.c_uint64]
            L.orc_reduce.restype = C.c_uint64
            L.orc_reduce.argtypes = [C.c_uint64, C.c_int64]
            L.orc_sigridhash.restype = C.c_int64
            L.orc_sigridhash.argtypes = [C.c_int64, C.c_uint64, C.c_int64]
            L.orc_logit.restype = C.c_float
            L.orc_logit.argtypes = [C.c_float, C.c_float]
            L.orc_boxcox.restype = C.c_float
            L.orc_boxcox.argtypes = [C.c_float, C.c_float]
            L.orc_bucketize_f.restype = C.c_int64
            L.orc_bucketize_f.argtypes = [C.c_float, C.c_void_p, C.c_int32]
            L.orc_bucketize_i.restype = C.c_int64
            L.orc_bucketize_i.argtypes = [C.c_int64, C.c_void_p, C.c_int32]
            L.orc_ngram.restype = C.c_int64
            L.orc_ngram.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_uint64, C.c_int64, C.c_void_p]
            L.orc_validate.restype = C.c_int
            L.orc_validate.argtypes = [C.POINTER(OrcGraph), C.POINTER(C.c_int64), C.POINTER(C.c_int64)]
            L.orc_run.restype = C.c_int
            L.orc_run.argtypes = [C.POINTER(OrcGraph), C.POINTER(OrcBatch), C.POINTER(OrcResult)]
            L.orc_free.restype = None
            L.orc_free.argtypes = [C.POINTER(OrcResult)]
            _lib = L
    return _lib


# ---------------------------------------------------------------- scalar helpers
def H(x: int) -> int:
    return lib().orc_H(x & (2**64 - 1))


def reduce(h: int, M: int) -> int:
    return lib().orc_reduce(h & (2**64 - 1), M)


def sigridhash(x: int, salt: int, M: int) -> int:
    return lib().orc_sigridhash(x, salt & (2**64 - 1), M)


def logit(x: float, eps: float) -> float:
    return lib().orc_logit(x, eps)


def boxcox(x: float, lam: float) -> float:
    return lib().orc_boxcox(x, lam)


def bucketize_f(x: float, borders) -> int:
    b = np.ascontiguousarray(borders, dtype=np.float32)
    return lib().orc_bucketize_f(x, b.ctypes.data, len(b))


def bucketize_i(x: int, borders) -> int:
    b = np.ascontiguousarray(borders, dtype=np.int64)
    return lib().orc_bucketize_i(x, b.ctypes.data, len(b))


def ngram(ids, n: int, salt: int, M: int):
    c = np.ascontiguousarray(ids, dtype=np.int64)
    out = np.zeros(max(len(c), 1), dtype=np.int64)
    cnt = lib().orc_ngram(c.ctypes.data, len(c), n, salt & (2**64 - 1), M, out.ctypes.data)
    return [int(v) for v in out[:cnt]]


# ---------------------------------------------------------------- graph marshalling
def _graph(spec):
    """Build OrcGraph from a graph-spec dict; returns (graph, keepalive)."""
    keep = []
    nodes = spec["nodes"]
    arr = (OrcNode * max(len(nodes), 1))()
    for i, nd in enumerate(nodes):
        o = arr[i]
        o.op = OPS[nd["op"]] if isinstance(nd["op"], str) else int(nd["op"])
        ins = nd["inputs"]
        o.n_in = len(ins)
        for j, (kind, idx) in enumerate(ins[:MAX_IN]):
            o.in_kind[j] = IN_KIND[kind]
            o.in_idx[j] = idx
        o.f_fill = nd.get("f_fill", 0.0)
        o.eps = nd.get("eps", 1e-6)
        o.lam = nd.get("lambda", 0.0)
        o.i_fill = nd.get("i_fill", 0)
        o.lo = nd.get("lo", 0)
        o.hi = nd.get("hi", 0)
        o.x = nd.get("x", 0)
        o.max_value = nd.get("max_value", 0)
        o.map_default = nd.get("map_default", 0)
        o.salt = nd.get("salt", 0) & (2**64 - 1)
        o.n = nd.get("n", 0)
        o.k_width = nd.get("k", 0)
        if "borders" in nd:
            b = np.asarray(nd["borders"])
            o.n_borders = nd.get("n_borders", len(b))
            fb = np.ascontiguousarray(b, dtype=np.float32)
            ib = np.ascontiguousarray(b if b.dtype.kind in "iu" else np.zeros(len(b)), dtype=np.int64)
            keep += [fb, ib]
            o.f_borders = fb.ctypes.data if len(fb) else None
            o.i_borders = ib.ctypes.data if len(ib) else None
        else:
            o.n_borders = nd.get("n_borders", 0)
        if "keys" in nd:
            k = np.ascontiguousarray(nd["keys"], dtype=np.int64)
            v = np.ascontiguousarray(nd["vals"], dtype=np.int64)
            keep += [k, v]
            o.map_size = nd.get("map_size", len(k))
            o.map_keys = k.ctypes.data if len(k) else None
            o.map_vals = v.ctypes.data if len(v) else None
        else:
            o.map_size = nd.get("map_size", 0)
    outs = (C.c_int32 * max(len(spec["outputs"]), 1))(*spec["outputs"])
    g = OrcGraph(spec["n_dense"], spec["n_sparse"], len(nodes), arr, len(spec["outputs"]), outs)
    keep += [arr, outs]
    return g, keep


def validate(spec):
    g, keep = _graph(spec)
    d, f = C.c_int64(), C.c_int64()
    st = lib().orc_validate(C.byref(g), C.byref(d), C.byref(f))
    return STATUS.get(st, str(st)), d.value, f.value


def _ptrs(arrs):
    a = (C.c_void_p * max(len(arrs), 1))()
    for i, x in enumerate(arrs):
        a[i] = None if x is None else x.ctypes.data
    return a


def run(spec, batch):
    """Run the oracle on a host batch (dict of numpy arrays, see synth.Batch).

    Returns dict(status, dense[B, D], lengths[F*B], offsets[F*B+1], values[N]).
    """
    g, keep = _graph(spec)
    dense = [np.ascontiguousarray(x, dtype=np.float32) for x in batch["dense"]]
    dval = [None if x is None else np.ascontiguousarray(x, dtype=np.uint32) for x in batch["dense_valid"]]
    soff = [np.ascontiguousarray(x, dtype=np.int32) for x in batch["sp_off"]]
    sval = [np.ascontiguousarray(x, dtype=np.int64) for x in batch["sp_val"]]
    svld = [None if x is None else np.ascontiguousarray(x, dtype=np.uint32) for x in batch["sp_valid"]]
    keep += [dense, dval, soff, sval, svld]
    P = [_ptrs(dense), _ptrs(dval), _ptrs(soff), _ptrs(sval), _ptrs(svld)]
    keep += P
    b = OrcBatch(int(batch["n_rows"]), *P)
    r = OrcResult()
    st = lib().orc_run(C.byref(g), C.byref(b), C.byref(r))
    if st != 0:
        return {"status": STATUS.get(st, str(st))}
    B, D, F, N = r.n_rows, r.d_out, r.f_out, r.n_values
    out = {
        "status": "OK",
        "dense": np.ctypeslib.as_array(r.dense, shape=(max(B * D, 1),))[: B * D].copy().reshape(B, D),
        "lengths": np.ctypeslib.as_array(r.lengths, shape=(max(B * F, 1),))[: B * F].copy(),
        "offsets": np.ctypeslib.as_array(r.offsets, shape=(B * F + 1,)).copy(),
        "values": np.ctypeslib.as_array(r.values, shape=(max(N, 1),))[:N].copy(),
    }
    lib().orc_free(C.byref(r))
    return out
