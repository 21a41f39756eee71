#!/usr/bin/env python
"""compute-sanitizer driver: C1 / C2 / multi-hot / random
batches through every fused kernel, with every input column and validity
bitmap in its own cudaMalloc of EXACTLY its size (ceil(B/32) words for a
bitmap, B+1 offsets, nnz ids), so memcheck flags any read past a column.
Outputs are also compared with the oracle (a sanitizer run must not change
values).  Run as:
  compute-sanitizer --tool memcheck python scripts/sanitize.py
  compute-sanitizer --tool racecheck python scripts/sanitize.py
"""
import ctypes as C
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from oracle import oracle  # noqa: E402
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402
from tests.parity import assert_parity  # noqa: E402

_rt = C.CDLL("/usr/local/cuda/lib64/libcudart.so.12")
_rt.cudaMalloc.argtypes = [C.POINTER(C.c_void_p), C.c_size_t]
_rt.cudaMemcpy.argtypes = [C.c_void_p, C.c_void_p, C.c_size_t, C.c_int]
_rt.cudaFree.argtypes = [C.c_void_p]


class Exact:
    """A device copy of a host array in a cudaMalloc of exactly its bytes."""

    def __init__(self, a):
        a = np.ascontiguousarray(a)
        self.nbytes = max(a.nbytes, 1)
        self.p = C.c_void_p()
        assert _rt.cudaMalloc(C.byref(self.p), self.nbytes) == 0
        if a.nbytes:
            assert _rt.cudaMemcpy(self.p, a.ctypes.data, a.nbytes, 1) == 0

    def data_ptr(self):
        return self.p.value

    def __del__(self):
        _rt.cudaFree(self.p)


class ExactBatch(rap.DeviceBatch):
    def __init__(self, batch):  # noqa: D401 - same fields as DeviceBatch, exact allocations
        self.n_rows = int(batch["n_rows"])
        self.dense = [Exact(np.asarray(x, np.float32)) for x in batch["dense"]]
        self.dense_valid = [None if x is None else Exact(np.asarray(x, np.uint32)) for x in batch["dense_valid"]]
        self.sp_off = [Exact(np.asarray(x, np.int32)) for x in batch["sp_off"]]
        self.sp_val = [Exact(np.asarray(x, np.int64)) for x in batch["sp_val"]]
        self.sp_valid = [None if x is None else Exact(np.asarray(x, np.uint32)) for x in batch["sp_valid"]]
        self.sp_nnz = np.array([int(o[-1]) - int(o[0]) for o in batch["sp_off"]] or [0], dtype=np.int64)
        for v, o in zip(self.dense_valid + self.sp_valid, list(batch["dense_valid"]) + list(batch["sp_valid"])):
            if v is not None:
                assert v.nbytes == 4 * ((self.n_rows + 31) // 32) == np.asarray(o).nbytes
        self._build_struct()


def cases():
    from tests.test_gpu_parity import _random_graph

    yield "c2", synth.c2_terabyte(0).spec, synth.make_batch(synth.c2_terabyte(0), 3000, seed=3)
    yield "c1", synth.c1_kaggle(0).spec, synth.make_batch(synth.c1_kaggle(0), 1001, seed=4)
    w = synth.c4_multihot(0, n_features=24)
    yield "multihot", w.spec, synth.make_batch(w, 2020, seed=5)
    from tests.helpers import batch

    for seed in range(2):  # the random-graph recipe of tests/test_gpu_parity.py
        rng = np.random.default_rng(100 + seed)
        s = _random_graph(rng, 3, 4)
        B = int(rng.integers(500, 4000))
        dense = [synth.dense_column(seed, c, "unit" if c % 2 else "count", B) for c in range(3)]
        means = [None, 3.0, 0.5, 12.0]
        sparse = [synth.sparse_column(seed, sc, 5000, B, means[sc], null_p=0.15, null_segments=(sc == 2),
                                      base_offset=sc) for sc in range(4)]
        yield f"random{seed}", s, batch(B, dense=dense, sparse=sparse)


def main():
    rap.load()
    modes = [int(m) for m in os.environ.get("KMODES", "1,2,3").split(",")]
    only = [c for c in os.environ.get("CASES", "").split(",") if c]
    n = 0
    for name, spec, host in cases():
        if only and name not in only:
            continue
        want = oracle.run(spec, host)
        for km in modes:
            plan = rap.Plan(spec, device=0)
            plan.set_kernel(km)
            raw = ExactBatch(host)
            out = rap.DeviceOutput(plan, host["n_rows"], raw.sp_nnz, "cuda:0")
            plan.preprocess(raw, out)
            plan.preprocess(raw, out)  # second launch: counters reset by the last CTA
            torch.cuda.synchronize()
            assert plan.check_overflow() == 0
            assert_parity(out.to_numpy(), want, ctx=f"{name} kernel {km}")
            plan.close()
            n += 1
            print(f"{name} kernel {km}: ok", flush=True)
    print(f"sanitize: {n} launches pairs ok")


if __name__ == "__main__":
    main()
