#!/usr/bin/env python
"""Warm up and run a few launches of one workload (target for ncu captures; dev tool)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402

wl = os.environ.get("WL", "c2")
w = {"c2": synth.c2_terabyte, "c1": synth.c1_kaggle, "c4": synth.c4_multihot}[wl](0)
B = int(os.environ.get("B", "65536"))
plan = rap.Plan(w.spec, device=0)
if os.environ.get("KMODE"):
    plan.set_kernel(int(os.environ["KMODE"]))
h = synth.make_batch(w, B, seed=1000)
r = rap.DeviceBatch(h, "cuda:0")
o = rap.DeviceOutput(plan, B, r.sp_nnz, "cuda:0")
for _ in range(int(os.environ.get("N", "3"))):
    plan.preprocess(r, o)
torch.cuda.synchronize()
print("ok", plan.info().get("grid"))
