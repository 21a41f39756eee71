#!/usr/bin/env python
"""Launches of the C2 plan at one SM budget (env BUDGET, KMODE) for an ncu
capture of the kernel's SM footprint (dev tool):
  ncu --metrics sm__cycles_active.sum,sm__cycles_active.max,... python scripts/budget_footprint.py"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402


def main():
    w = synth.c2_terabyte(0)
    B = int(os.environ.get("B", "65536"))
    h = synth.make_batch(w, B, seed=5)
    budget = int(os.environ.get("BUDGET", "0"))
    part = None
    if os.environ.get("PART") == "1":  # a green-context SM partition of `budget` SMs
        part = rap.SMPartitionStream(0, budget)
        budget = part.sms
        print("partition SMs", part.sms)
    plan = rap.Plan(w.spec, device=0, sm_budget=budget)
    plan.set_kernel(int(os.environ.get("KMODE", "0")))
    raw = rap.DeviceBatch(h, "cuda:0")
    out = rap.DeviceOutput(plan, B, raw.sp_nnz, "cuda:0")
    st = part.stream if part else torch.cuda.current_stream()
    for _ in range(3):
        plan.preprocess(raw, out, st)
    torch.cuda.synchronize()
    if part:
        part.close()
    print("grid", plan.info()["grid"], "kernel", plan.info()["kernel_last"])
    plan.close()


if __name__ == "__main__":
    main()
