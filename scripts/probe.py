#!/usr/bin/env python
"""Time sub-graphs of the C2 workload to attribute kernel time (dev tool)."""
import copy
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402


def subspec(spec, keep_outputs):
    s = copy.deepcopy(spec)
    s["outputs"] = keep_outputs
    return s


def time_spec(spec, host, steps=200, budget=0):
    plan = rap.Plan(spec, device=0, sm_budget=budget)
    raws = [rap.DeviceBatch(host, "cuda:0") for _ in range(4)]
    outs = [rap.DeviceOutput(plan, host["n_rows"], raws[0].sp_nnz, "cuda:0") for _ in range(4)]
    for i in range(10):
        plan.preprocess(raws[i % 4], outs[i % 4])
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(steps):
        plan.preprocess(raws[i % 4], outs[i % 4])
    e1.record()
    e1.synchronize()
    info = plan.info()
    plan.close()
    return e0.elapsed_time(e1) / steps * 1e3, info


def main():
    w = synth.c2_terabyte(0)
    B = int(os.environ.get("B", "65536"))
    host = synth.make_batch(w, B, seed=1)
    outs = w.spec["outputs"]
    dense_outs = outs[:15]
    sparse_outs = outs[15:41]
    ngram_outs = outs[41:]
    plain = [o for i, o in enumerate(sparse_outs) if i not in (1, 5, 9, 13, 17, 21, 3, 11, 19, 24)]
    cases = {
        "full": outs,
        "dense(15 units)": dense_outs,
        "sparse26": sparse_outs,
        "sparse16 clamp+hash": plain,
        "ngram8": ngram_outs,
        "one sparse feature": sparse_outs[:1],
        "one ngram": ngram_outs[:1],
    }
    for name, keep in cases.items():
        us, info = time_spec(subspec(w.spec, keep), host)
        print(f"{name:24s} {us:9.2f} us   grid {info['grid']} desc {info['n_descriptors_last']}", flush=True)


if __name__ == "__main__":
    main()
