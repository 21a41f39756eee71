"""Thin ctypes binding of librap.so (include/rap.h).

Argument marshalling only: every step of the preprocessing path runs in the
CUDA kernel behind the C ABI.  PyTorch supplies device memory and streams.
There is no fallback: if librap.so is missing this module raises on import
of the library (``load()``), and nothing here computes any operator.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import _build

OPS = {"fillnull": 0, "logit": 1, "boxcox": 2, "onehot": 3, "sigridhash": 4,
       "bucketize": 5, "firstx": 6, "clamp": 7, "ngram": 8, "mapid": 9}
STATUS = {0: "OK", 1: "INVALID_ARGUMENT", 2: "INVALID_GRAPH", 3: "INVALID_PARAM", 4: "CAPACITY",
          5: "UNSUPPORTED", 6: "CUDA", 7: "OUT_OF_MEMORY"}

EXPORTS = ["rap_plan_create", "rap_plan_output_shape", "rap_preprocess", "rap_preprocess_host", "rap_preprocess_host_async", "rap_set_budget",
           "rap_predict_latency_us", "rap_choose_budget", "rap_plan_info_get", "rap_debug_trace", "rap_plan_destroy",
           "rap_status_string", "rap_last_error", "rap_shard_rows", "rap_plan_output_costs", "rap_place",
           "rap_plan_create_sharded", "rap_jagged_append", "rap_set_kernel", "rap_check_overflow",
           "rap_debug_jit_source", "rap_place_comm", "rap_place_joint", "rap_predict_terms", "rap_sm_partition_stream",
           "rap_sm_partition_stream_destroy"]
PLACE_MODES = {"balanced": 0, "round_robin": 1, "skewed": 2}
RAP_OUT_CHAIN = 1


class RapError(RuntimeError):
    def __init__(self, status, detail=""):
        self.status = STATUS.get(status, str(status))
        super().__init__(f"RAP_ERR_{self.status}: {detail}")


class RapNode(C.Structure):
    _fields_ = [("op", C.c_int32), ("n_inputs", C.c_int32), ("inputs", C.POINTER(C.c_int32)), ("param", C.c_int32)]


class RapGraph(C.Structure):
    _fields_ = [("n_dense_in", C.c_int32), ("n_sparse_in", C.c_int32), ("n_nodes", C.c_int32),
                ("nodes", C.POINTER(RapNode)), ("n_outputs", C.c_int32), ("output_nodes", C.POINTER(C.c_int32))]


class RapOpParam(C.Structure):
    _fields_ = [("f_fill", C.c_float), ("eps", C.c_float), ("lam", C.c_float),
                ("i_fill", C.c_int64), ("lo", C.c_int64), ("hi", C.c_int64), ("x", C.c_int64),
                ("max_value", C.c_int64), ("map_default", C.c_int64), ("salt", C.c_uint64),
                ("n", C.c_int32), ("k_width", C.c_int32), ("n_borders", C.c_int32), ("borders", C.c_void_p),
                ("map_size", C.c_int64), ("map_keys", C.c_void_p), ("map_vals", C.c_void_p)]


class RapRawBatch(C.Structure):
    _fields_ = [("n_rows", C.c_int64), ("dense", C.c_void_p), ("dense_valid", C.c_void_p),
                ("sp_offsets", C.c_void_p), ("sp_values", C.c_void_p), ("sp_valid", C.c_void_p),
                ("sp_nnz", C.c_void_p)]


class RapOutput(C.Structure):
    _fields_ = [("dense_out", C.c_void_p), ("dense_ld", C.c_int64), ("lengths", C.c_void_p),
                ("offsets", C.c_void_p), ("values", C.c_void_p), ("values_capacity", C.c_int64),
                ("flags", C.c_int32), ("reserved", C.c_int32)]


class RapResidual(C.Structure):
    _fields_ = [("output", C.c_int32), ("owner", C.c_int32), ("helper", C.c_int32), ("pad", C.c_int32),
                ("split_row", C.c_int64)]


class RapCommModel(C.Structure):
    _fields_ = [("us_per_unit", C.c_double), ("link_gbs", C.c_double), ("link_latency_us", C.c_double),
                ("row_bytes", C.c_void_p)]


class RapPlanInfo(C.Structure):
    _fields_ = [("device", C.c_int32), ("sm_count", C.c_int32), ("sm_budget", C.c_int32),
                ("ctas_per_sm", C.c_int32), ("threads_per_cta", C.c_int32), ("grid", C.c_int32),
                ("n_dense_out_cols", C.c_int32), ("n_sparse_out", C.c_int32), ("n_dense_groups", C.c_int32),
                ("rows_per_dense_desc", C.c_int32), ("max_rows_per_sparse_desc", C.c_int32),
                ("min_rows_per_sparse_desc", C.c_int32), ("n_descriptors_last", C.c_int64),
                ("n_launches", C.c_int64), ("smem_bytes", C.c_int64),
                ("kernel_mode", C.c_int32), ("kernel_last", C.c_int32), ("rows_ctas_per_sm", C.c_int32),
                ("rows_smem_bytes", C.c_int32), ("rb_row_blocks", C.c_int32), ("rb_feature_groups", C.c_int32),
                ("rb_rows", C.c_int32), ("rb_memo_slots", C.c_int32), ("partition_uploads", C.c_int64),
                ("jit_state", C.c_int32), ("jit_ctas_per_sm", C.c_int32), ("jit_compile_seconds", C.c_double)]


# rap_set_kernel modes (include/rap.h).  DEFAULT_KERNEL is applied to every new
# Plan (env RAP_KERNEL; tests set it to run each parity case on both kernels).
KERNEL_AUTO, KERNEL_TILED, KERNEL_ROWS, KERNEL_JIT = 0, 1, 2, 3
OUT_CHAIN, OUT_VALUES_I32 = 1, 2  # rap_output.flags (include/rap.h)
DEFAULT_KERNEL = int(os.environ.get("RAP_KERNEL", "0"))


_lib = None


def load(build_if_stale: bool = False):
    """Load librap.so.  Raises if it is missing — there is no fallback path."""
    global _lib
    if _lib is not None:
        return _lib
    if build_if_stale:
        _build.build()
    if not os.path.exists(_build.LIB):
        raise ImportError(f"librap.so not built at {_build.LIB}; run __graft_entry__.build()")
    L = C.CDLL(_build.LIB)
    P = C.c_void_p
    L.rap_plan_create.restype = C.c_int
    L.rap_plan_create.argtypes = [C.POINTER(RapGraph), C.POINTER(RapOpParam), C.c_int32, C.c_int32, C.c_int32,
                                  C.POINTER(P)]
    L.rap_plan_output_shape.restype = C.c_int
    L.rap_plan_output_shape.argtypes = [P, C.c_int64, P, C.POINTER(C.c_int64), C.POINTER(C.c_int64),
                                        C.POINTER(C.c_int64)]
    L.rap_preprocess.restype = C.c_int
    L.rap_preprocess.argtypes = [P, C.POINTER(RapRawBatch), C.POINTER(RapOutput), P]
    L.rap_preprocess_host.restype = C.c_int
    L.rap_preprocess_host.argtypes = [P, C.POINTER(RapRawBatch), C.POINTER(RapOutput), P]
    L.rap_preprocess_host_async.restype = C.c_int
    L.rap_preprocess_host_async.argtypes = [P, C.POINTER(RapRawBatch), C.POINTER(RapOutput), P]
    L.rap_set_budget.restype = C.c_int
    L.rap_set_budget.argtypes = [P, C.c_int32]
    L.rap_predict_latency_us.restype = C.c_int
    L.rap_predict_latency_us.argtypes = [P, C.c_int64, P, C.c_int32, C.POINTER(C.c_double)]
    L.rap_predict_terms.restype = C.c_int
    L.rap_predict_terms.argtypes = [P, C.c_int64, P, C.c_int32, P]
    L.rap_sm_partition_stream.restype = C.c_int
    L.rap_sm_partition_stream.argtypes = [C.c_int32, C.c_int32, C.c_int32, C.POINTER(P), C.POINTER(C.c_int32)]
    L.rap_sm_partition_stream_destroy.restype = C.c_int
    L.rap_sm_partition_stream_destroy.argtypes = [P]
    L.rap_choose_budget.restype = C.c_int
    L.rap_choose_budget.argtypes = [P, C.c_int64, P, C.c_double, C.POINTER(C.c_int32), C.POINTER(C.c_double)]
    L.rap_plan_info_get.restype = C.c_int
    L.rap_plan_info_get.argtypes = [P, C.POINTER(RapPlanInfo)]
    L.rap_set_kernel.restype = C.c_int
    L.rap_set_kernel.argtypes = [P, C.c_int32]
    L.rap_check_overflow.restype = C.c_int
    L.rap_check_overflow.argtypes = [P, C.POINTER(C.c_int32)]
    L.rap_debug_jit_source.restype = C.c_int
    L.rap_debug_jit_source.argtypes = [C.POINTER(RapGraph), C.POINTER(RapOpParam), C.c_int32, C.c_char_p, C.c_int64,
                                       C.c_int32, C.POINTER(C.c_int32)]
    L.rap_debug_trace.restype = C.c_int
    L.rap_debug_trace.argtypes = [P, C.c_int32, P, C.c_int64, C.POINTER(C.c_int64)]
    L.rap_plan_destroy.restype = None
    L.rap_plan_destroy.argtypes = [P]
    L.rap_status_string.restype = C.c_char_p
    L.rap_status_string.argtypes = [C.c_int]
    L.rap_last_error.restype = C.c_char_p
    L.rap_last_error.argtypes = []
    L.rap_shard_rows.restype = C.c_int
    L.rap_shard_rows.argtypes = [C.c_int64, C.c_int32, C.c_int32, C.POINTER(C.c_int64), C.POINTER(C.c_int64)]
    L.rap_plan_output_costs.restype = C.c_int
    L.rap_plan_output_costs.argtypes = [P, C.c_int64, P, P]
    L.rap_place.restype = C.c_int
    L.rap_place.argtypes = [P, P, C.c_int32, C.c_int32, C.c_int32, C.c_int64, C.c_double, P, P,
                            C.POINTER(RapResidual)]
    L.rap_place_comm.restype = C.c_int
    L.rap_place_comm.argtypes = [P, P, C.c_int32, C.c_int32, C.c_int32, C.c_int64, C.POINTER(RapCommModel), P, P,
                                 C.POINTER(RapResidual)]
    L.rap_place_joint.restype = C.c_int
    L.rap_place_joint.argtypes = [P, P, P, C.c_int32, C.c_int32, C.c_int64, C.POINTER(RapCommModel), C.c_double, P, P,
                                  C.POINTER(C.c_int32)]
    L.rap_plan_create_sharded.restype = C.c_int
    L.rap_plan_create_sharded.argtypes = [C.POINTER(RapGraph), C.POINTER(RapOpParam), C.c_int32, C.c_int32, C.c_int32,
                                          P, C.c_int32, C.c_int32, C.POINTER(P)]
    L.rap_jagged_append.restype = C.c_int
    L.rap_jagged_append.argtypes = [P, P, P, C.c_int64, C.c_int64, P, P, P, C.c_int64, P]
    _lib = L
    return L


def _check(st):
    if st != 0:
        raise RapError(st, load().rap_last_error().decode())


def raw_ref(kind: str, idx: int) -> int:
    if kind == "n":
        return int(idx)
    if kind == "d":
        return -1 - 2 * int(idx)
    return -2 - 2 * int(idx)


def marshal_graph(spec):
    """Graph-spec dict (synth.py docstring) -> (RapGraph, RapOpParam[], keepalive)."""
    keep = []
    nodes = spec["nodes"]
    n = len(nodes)
    cn = (RapNode * max(n, 1))()
    cp = (RapOpParam * max(n, 1))()
    for i, nd in enumerate(nodes):
        ins = (C.c_int32 * max(len(nd["inputs"]), 1))(*[raw_ref(k, x) for k, x in nd["inputs"]])
        keep.append(ins)
        op = nd["op"]
        cn[i].op = OPS[op] if isinstance(op, str) else int(op)
        cn[i].n_inputs = len(nd["inputs"])
        cn[i].inputs = ins
        cn[i].param = i
        p = cp[i]
        p.f_fill = nd.get("f_fill", 0.0)
        p.eps = nd.get("eps", 1e-6)
        p.lam = nd.get("lambda", 0.0)
        p.i_fill = nd.get("i_fill", 0)
        p.lo = nd.get("lo", 0)
        p.hi = nd.get("hi", 0)
        p.x = nd.get("x", 0)
        p.max_value = nd.get("max_value", 0)
        p.map_default = nd.get("map_default", 0)
        p.salt = nd.get("salt", 0) & (2**64 - 1)
        p.n = nd.get("n", 0)
        p.k_width = nd.get("k", 0)
        if "borders" in nd:
            b = np.asarray(nd["borders"])
            arr = np.ascontiguousarray(b, dtype=np.int64 if b.dtype.kind in "iu" else np.float32)
            keep.append(arr)
            p.n_borders = nd.get("n_borders", len(arr))
            p.borders = arr.ctypes.data if len(arr) else None
        else:
            p.n_borders = nd.get("n_borders", 0)
        if "keys" in nd:
            k = np.ascontiguousarray(nd["keys"], dtype=np.int64)
            v = np.ascontiguousarray(nd["vals"], dtype=np.int64)
            keep += [k, v]
            p.map_size = nd.get("map_size", len(k))
            p.map_keys = k.ctypes.data if len(k) else None
            p.map_vals = v.ctypes.data if len(v) else None
        else:
            p.map_size = nd.get("map_size", 0)
    outs = (C.c_int32 * max(len(spec["outputs"]), 1))(*spec["outputs"])
    g = RapGraph(spec["n_dense"], spec["n_sparse"], n, cn, len(spec["outputs"]), outs)
    keep += [cn, cp, outs]
    return g, cp, keep


def _ptr_array(ptrs):
    a = (C.c_void_p * max(len(ptrs), 1))()
    for i, x in enumerate(ptrs):
        a[i] = x
    return a


def _stream_handle(stream):
    if stream is None:
        import torch

        return C.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return C.c_void_p(stream)
    return C.c_void_p(stream.cuda_stream)


class DeviceBatch:
    """A raw batch resident in device memory (torch tensors) + its C struct."""

    def __init__(self, batch, device, pin=False, sparse_cols=None, dense_rows=None):
        """sparse_cols: upload only these raw sparse columns (the others get
        NULL pointers: a sharded rank's plan reads only its own tables'
        columns).  dense_rows = (row0, n): upload only those dense rows (a
        rank's batch shard, row0 a multiple of 128); the column pointers are
        biased by -row0 so the kernel's global row indices land in the copy."""
        import torch

        self.n_rows = int(batch["n_rows"])
        dev = torch.device(device) if not pin else torch.device("cpu")

        def t(a, dt):
            x = torch.from_numpy(np.ascontiguousarray(a, dtype=dt))
            return x.pin_memory() if pin else x.to(dev, non_blocking=False)

        r0, nd = (0, self.n_rows) if dense_rows is None else dense_rows
        assert r0 % 128 == 0 and 0 <= r0 and r0 + nd <= self.n_rows
        self._dense_bias = r0
        self.dense = [t(x[r0:r0 + nd], np.float32) for x in batch["dense"]]
        w0, w1 = r0 // 32, (r0 + nd + 31) // 32
        self.dense_valid = [None if x is None else t(x[w0:w1], np.uint32) for x in batch["dense_valid"]]
        keep = range(len(batch["sp_off"])) if sparse_cols is None else set(sparse_cols)
        self.sp_off = [t(x, np.int32) if c in keep else None for c, x in enumerate(batch["sp_off"])]
        self.sp_val = [(t(x, np.int64) if len(x) else t(np.zeros(1, np.int64), np.int64)) if c in keep else None
                       for c, x in enumerate(batch["sp_val"])]
        self.sp_valid = [None if (x is None or c not in keep) else t(x, np.uint32)
                         for c, x in enumerate(batch["sp_valid"])]
        self.sp_nnz = np.array([int(o[-1]) - int(o[0]) for o in batch["sp_off"]] or [0], dtype=np.int64)
        self._build_struct()

    def uploaded_bytes(self) -> int:
        xs = self.dense + self.dense_valid + self.sp_off + self.sp_val + self.sp_valid
        return int(sum(x.numel() * x.element_size() for x in xs if x is not None))

    def _build_struct(self):
        def ptr(x):
            return None if x is None else x.data_ptr()

        bias = getattr(self, "_dense_bias", 0)

        def dptr(x, elem_rows):  # dense pointers biased to global row 0 (dense_rows shard uploads)
            return None if x is None else x.data_ptr() - (bias // elem_rows) * 4

        self._arrs = [_ptr_array([dptr(x, 1) for x in self.dense]),
                      _ptr_array([dptr(x, 32) for x in self.dense_valid]),
                      _ptr_array([ptr(x) for x in self.sp_off]), _ptr_array([ptr(x) for x in self.sp_val]),
                      _ptr_array([ptr(x) for x in self.sp_valid])]
        a = self._arrs
        self.struct = RapRawBatch(self.n_rows, C.cast(a[0], C.c_void_p), C.cast(a[1], C.c_void_p),
                                  C.cast(a[2], C.c_void_p), C.cast(a[3], C.c_void_p), C.cast(a[4], C.c_void_p),
                                  self.sp_nnz.ctypes.data)


def row_view(raw: "DeviceBatch", row0: int, n_rows: int) -> "RapRawBatch":
    """A RapRawBatch over rows [row0, row0 + n_rows) of a device batch (pointer
    arithmetic only; row0 a multiple of 32 so validity words stay whole).
    sp_nnz stays the full batch's (an upper bound, used only for capacity)."""
    assert row0 % 32 == 0 and 0 <= row0 and row0 + n_rows <= raw.n_rows
    bias = getattr(raw, "_dense_bias", 0)  # a dense_rows upload holds rows [bias, ...)

    def ptrs(xs, elem, scale=1, b=0):
        return _ptr_array([None if x is None else x.data_ptr() + ((row0 - b) // scale) * elem for x in xs])
    arrs = [ptrs(raw.dense, 4, 1, bias), ptrs(raw.dense_valid, 4, 32, bias), ptrs(raw.sp_off, 4),
            _ptr_array([None if x is None else x.data_ptr() for x in raw.sp_val]), ptrs(raw.sp_valid, 4, 32)]
    st = RapRawBatch(n_rows, *[C.cast(a, C.c_void_p) for a in arrs], raw.sp_nnz.ctypes.data)
    st._keep = arrs
    return st


class DeviceOutput:
    """Output tensors (device, or pinned host when pin=True) + their C struct."""

    def __init__(self, plan, n_rows, sp_nnz, device, pin=False, dense_ld=None, capacity=None, values_i32=False):
        """values_i32: the ids emitted as int32 (Cast, RAP_OUT_VALUES_I32)."""
        import torch

        d, f, vb = plan.output_shape(n_rows, sp_nnz)
        self.d_out, self.f_out, self.bound = d, f, vb
        ld = d if dense_ld is None else dense_ld
        kw = {"pin_memory": True} if pin else {"device": device}
        self.dense = torch.empty(max(n_rows * ld, 1), dtype=torch.float32, **kw)
        self.lengths = torch.empty(max(n_rows * f, 1), dtype=torch.int32, **kw)
        self.offsets = torch.empty(n_rows * f + 1, dtype=torch.int64, **kw)
        cap = vb if capacity is None else capacity
        self.values = torch.empty(max(cap, 1), dtype=torch.int32 if values_i32 else torch.int64, **kw)
        self.n_rows, self.ld = n_rows, ld
        self.struct = RapOutput(self.dense.data_ptr(), ld, self.lengths.data_ptr(), self.offsets.data_ptr(),
                                self.values.data_ptr(), cap)
        if values_i32:
            self.struct.flags = OUT_VALUES_I32

    def to_numpy(self):
        B, d, f = self.n_rows, self.d_out, self.f_out
        off = self.offsets.cpu().numpy()
        n = int(off[-1]) if len(off) else 0
        # only the written elements are read (never the capacity tail or the
        # ld padding columns: initcheck-clean)
        dense = self.dense[: B * self.ld].view(B, self.ld)[:, :d] if B * self.ld else self.dense[:0].view(B, d)
        return {"dense": dense.contiguous().cpu().numpy(),
                "lengths": self.lengths[: B * f].cpu().numpy(), "offsets": off,
                "values": self.values[:n].cpu().numpy()}


class Plan:
    """rap_plan_create / rap_preprocess / rap_set_budget (include/rap.h)."""

    def __init__(self, spec, device: int = 0, sm_budget: int = 0):
        L = load()
        self.spec = spec
        g, params, self._keep = marshal_graph(spec)
        h = C.c_void_p()
        _check(L.rap_plan_create(C.byref(g), params, len(spec["nodes"]), device, sm_budget, C.byref(h)))
        self.handle = h
        self.device = device
        if DEFAULT_KERNEL:
            self.set_kernel(DEFAULT_KERNEL)

    @classmethod
    def sharded(cls, spec, sparse_owner, rank: int, world: int, device: int = 0, sm_budget: int = 0):
        """rap_plan_create_sharded: this rank's sparse outputs (full batch) +
        every dense output over its batch shard (include/rap.h)."""
        L = load()
        self = cls.__new__(cls)
        self.spec = spec
        g, params, self._keep = marshal_graph(spec)
        own = np.ascontiguousarray(sparse_owner, dtype=np.int32)
        self._keep.append(own)
        h = C.c_void_p()
        _check(L.rap_plan_create_sharded(C.byref(g), params, len(spec["nodes"]), device, sm_budget,
                                         own.ctypes.data, rank, world, C.byref(h)))
        self.handle = h
        self.device = device
        if DEFAULT_KERNEL:
            self.set_kernel(DEFAULT_KERNEL)
        return self

    def output_costs(self, n_rows, sp_nnz):
        f = self.output_shape(n_rows, sp_nnz)[1]
        nnz = np.ascontiguousarray(sp_nnz if len(sp_nnz) else [0], dtype=np.int64)
        cost = np.zeros(max(f, 1), dtype=np.float64)
        _check(load().rap_plan_output_costs(self.handle, n_rows, nnz.ctypes.data, cost.ctypes.data))
        return cost[:f]

    def preprocess_struct(self, raw_struct, out_struct, stream=None):
        _check(load().rap_preprocess(self.handle, C.byref(raw_struct), C.byref(out_struct), _stream_handle(stream)))

    def close(self):
        if getattr(self, "handle", None):
            load().rap_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def output_shape(self, n_rows, sp_nnz):
        nnz = np.ascontiguousarray(sp_nnz if sp_nnz is not None and len(sp_nnz) else [0], dtype=np.int64)
        d, f, vb = C.c_int64(), C.c_int64(), C.c_int64()
        _check(load().rap_plan_output_shape(self.handle, n_rows, nnz.ctypes.data, C.byref(d), C.byref(f),
                                            C.byref(vb)))
        return d.value, f.value, vb.value

    def preprocess(self, raw: DeviceBatch, out: DeviceOutput, stream=None):
        _check(load().rap_preprocess(self.handle, C.byref(raw.struct), C.byref(out.struct), _stream_handle(stream)))

    def preprocess_host(self, raw: DeviceBatch, out: DeviceOutput, stream=None):
        """raw / out built with pin=True (host buffers); synchronises the stream."""
        _check(load().rap_preprocess_host(self.handle, C.byref(raw.struct), C.byref(out.struct),
                                          _stream_handle(stream)))

    def preprocess_host_async(self, raw: DeviceBatch, out: DeviceOutput, stream=None):
        """Host buffers (pin=True); enqueue only — sync the stream before reading out."""
        _check(load().rap_preprocess_host_async(self.handle, C.byref(raw.struct), C.byref(out.struct),
                                                _stream_handle(stream)))

    def set_budget(self, sm_budget: int):
        _check(load().rap_set_budget(self.handle, sm_budget))

    def set_kernel(self, mode: int):
        """rap_set_kernel: KERNEL_AUTO / KERNEL_TILED / KERNEL_ROWS."""
        _check(load().rap_set_kernel(self.handle, int(mode)))

    def check_overflow(self) -> int:
        """rap_check_overflow: 1 if a launch since the last query found more ids
        than values_capacity (synchronises the device; clears the flag)."""
        v = C.c_int32()
        _check(load().rap_check_overflow(self.handle, C.byref(v)))
        return v.value

    def info(self) -> dict:
        i = RapPlanInfo()
        _check(load().rap_plan_info_get(self.handle, C.byref(i)))
        return {k: getattr(i, k) for k, _ in RapPlanInfo._fields_}

    def trace_enable(self, cap: int):
        _check(load().rap_debug_trace(self.handle, 1, None, cap, None))

    def trace_read(self, cap: int):
        """Stamps of the last call: uint64 [n_cta, 24] (profiling aid)."""
        buf = np.zeros((cap, 24), dtype=np.uint64)
        n = C.c_int64()
        _check(load().rap_debug_trace(self.handle, 0, buf.ctypes.data, cap, C.byref(n)))
        return buf[: min(cap, n.value)]

    def trace_disable(self):
        _check(load().rap_debug_trace(self.handle, -1, None, 0, None))

    def predict_latency_us(self, n_rows, sp_nnz, sm_budget=0):
        nnz = np.ascontiguousarray(sp_nnz if len(sp_nnz) else [0], dtype=np.int64)
        v = C.c_double()
        _check(load().rap_predict_latency_us(self.handle, n_rows, nnz.ctypes.data, sm_budget, C.byref(v)))
        return v.value

    def predict_terms(self, n_rows, sp_nnz, sm_budget=0):
        """rap_predict_terms: (kernel, grid, busiest CTA's sparse work, bytes, its dense work, its pairs)."""
        nnz = np.ascontiguousarray(sp_nnz, dtype=np.int64)
        t = np.zeros(6, dtype=np.float64)
        _check(load().rap_predict_terms(self.handle, n_rows, nnz.ctypes.data, sm_budget, t.ctypes.data))
        return int(t[0]), int(t[1]), float(t[2]), float(t[3]), float(t[4]), float(t[5])

    def choose_budget(self, n_rows, sp_nnz, overlap_capacity_us):
        nnz = np.ascontiguousarray(sp_nnz if len(sp_nnz) else [0], dtype=np.int64)
        b, td = C.c_int32(), C.c_double()
        _check(load().rap_choose_budget(self.handle, n_rows, nnz.ctypes.data, overlap_capacity_us, C.byref(b),
                                        C.byref(td)))
        return b.value, td.value


class SMPartitionStream:
    """rap_sm_partition_stream: a CUDA stream (torch.cuda.ExternalStream) on a
    green-context partition of n_sms SMs (rounded up by the driver)."""

    def __init__(self, device: int, n_sms: int, priority: int = 0):
        import torch

        h, n = C.c_void_p(), C.c_int32()
        _check(load().rap_sm_partition_stream(device, n_sms, priority, C.byref(h), C.byref(n)))
        self.handle, self.sms = h.value, n.value
        self.stream = torch.cuda.ExternalStream(self.handle, device=torch.device("cuda", device))

    def close(self):
        if self.handle:
            self.stream.synchronize()
            _check(load().rap_sm_partition_stream_destroy(self.handle))
            self.handle = None


def jit_source(spec, compile: bool = False):
    """rap_debug_jit_source: the CUDA source the code generator emits for a
    spec (no device needed) and, with compile=True, whether NVRTC compiles it
    for sm_100a.  Returns (status name, source, compiled, nvrtc log)."""
    L = load()
    g, params, keep = marshal_graph(spec)
    cap = 1 << 22
    buf = C.create_string_buffer(cap)
    ok = C.c_int32(0)
    st = L.rap_debug_jit_source(C.byref(g), params, len(spec["nodes"]), buf, cap, 1 if compile else 0, C.byref(ok))
    return STATUS.get(st, str(st)), buf.value.decode(), bool(ok.value), L.rap_last_error().decode()


def validate_only(spec):
    """Status name rap_plan_create gives for a spec on device 0 (needs a GPU
    only when the graph is valid)."""
    L = load()
    g, params, keep = marshal_graph(spec)
    h = C.c_void_p()
    st = L.rap_plan_create(C.byref(g), params, len(spec["nodes"]), 0, 0, C.byref(h))
    if st == 0:
        L.rap_plan_destroy(h)
    return STATUS.get(st, str(st))
