#!/usr/bin/env python
"""Kernel time of one rap_preprocess vs SM budget (dev tool; calibrates the
co-running cost model rap_predict_latency_us).  Prints one JSON line per
(workload, budget) with the measured and the predicted microseconds."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402


def time_plan(plan, sets, steps=50):
    s = torch.cuda.current_stream()
    for i in range(5):
        plan.preprocess(sets[i % len(sets)][0], sets[i % len(sets)][1], s)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for i in range(steps):
        plan.preprocess(sets[i % len(sets)][0], sets[i % len(sets)][1], s)
    e1.record(s)
    e1.synchronize()
    return e0.elapsed_time(e1) / steps * 1e3


def main():
    budgets = [int(b) for b in os.environ.get("BUDGETS", "8,16,37,74,111,148").split(",")]
    cases = [("c1", synth.c1_kaggle(0), 4096), ("c1_1k", synth.c1_kaggle(0), 1024),
             ("c2", synth.c2_terabyte(0), 65536), ("c2_16k", synth.c2_terabyte(0), 16384),
             ("c2_4k", synth.c2_terabyte(0), 4096), ("c4_16k", synth.c4_multihot(0), 16384),
             ("c4_4k", synth.c4_multihot(0), 4096)]
    only = os.environ.get("CASES")
    if only:
        cases = [c for c in cases if c[0] in only.split(",")]
    for name, w, B in cases:
        plan = rap.Plan(w.spec, device=0)
        sets = []
        for i in range(3 if B <= 65536 else 2):
            h = synth.make_batch(w, B, seed=900 + i)
            r = rap.DeviceBatch(h, "cuda:0")
            sets.append((r, rap.DeviceOutput(plan, B, r.sp_nnz, "cuda:0")))
        nnz = sets[0][0].sp_nnz
        for b in budgets:
            plan.set_budget(b)
            us = time_plan(plan, sets, steps=20 if "c4" in name else 50)
            pred = plan.predict_latency_us(B, nnz, b)
            fam, grid, work, nbytes, dwork, pairs = plan.predict_terms(B, nnz, b)
            info = plan.info()
            print(json.dumps({"workload": name, "B": B, "budget": b, "measured_us": round(us, 2),
                              "predicted_us": round(pred, 2), "kernel": info["kernel_last"], "grid": info["grid"],
                              "model_kernel": fam, "model_grid": grid, "work": work, "bytes": nbytes,
                              "dwork": dwork, "pairs": pairs}),
                  flush=True)
        plan.close()
        del sets
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
