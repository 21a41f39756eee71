#!/usr/bin/env python
"""Fixed per-launch cost of rap_preprocess (dev tool): the kernel time at
several batch sizes, per call (events around each launch) and under CUDA-graph
replay, for a workload (WL=c1|c2).  The intercept at small B is the launch's
fixed cost."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402


def measure(plan, host, steps=400, nsets=4):
    B = host["n_rows"]
    raws = [rap.DeviceBatch(host, "cuda:0") for _ in range(nsets)]
    outs = [rap.DeviceOutput(plan, B, raws[0].sp_nnz, "cuda:0") for _ in range(nsets)]
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for i in range(20):
            plan.preprocess(raws[i % nsets], outs[i % nsets], stream=s)
    s.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        e0.record(s)
        for i in range(steps):
            plan.preprocess(raws[i % nsets], outs[i % nsets], stream=s)
        e1.record(s)
    e1.synchronize()
    per_call = e0.elapsed_time(e1) / steps * 1e3
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for i in range(nsets):
            plan.preprocess(raws[i], outs[i], stream=s)
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    reps = max(1, steps // nsets)
    e0.record()
    for _ in range(reps):
        g.replay()
    e1.record()
    e1.synchronize()
    graph = e0.elapsed_time(e1) / (reps * nsets) * 1e3
    return per_call, graph


def main():
    wl = os.environ.get("WL", "c1")
    w = {"c1": synth.c1_kaggle, "c2": synth.c2_terabyte, "c4": synth.c4_multihot}[wl](0)
    sizes = [int(x) for x in os.environ.get("SIZES", "32,128,1024,4096,16384,65536").split(",")]
    mode = os.environ.get("RAP_KERNEL_MODE")
    res = []
    for B in sizes:
        host = synth.make_batch(w, B, seed=3)
        plan = rap.Plan(w.spec, device=0)
        if mode is not None and hasattr(plan, "set_kernel"):
            plan.set_kernel(int(mode))
        pc, gr = measure(plan, host)
        info = plan.info()
        res.append({"B": B, "per_call_us": round(pc, 2), "graph_us": round(gr, 2), "grid": info["grid"]})
        print(f"{wl} B={B:6d} grid {info['grid']:4d}: per call {pc:8.2f} us   graph replay {gr:8.2f} us", flush=True)
        plan.close()
    print(json.dumps({"workload": wl, "mode": mode, "points": res}))


if __name__ == "__main__":
    main()
