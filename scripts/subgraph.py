#!/usr/bin/env python
"""Run a slice of the C2 graph's outputs a few times (for ncu; dev tool).
usage: KEEP=a:b python scripts/subgraph.py"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402

w = synth.c2_terabyte(0)
B = int(os.environ.get("B", "65536"))
host = synth.make_batch(w, B, seed=1)
spec = dict(w.spec)
a, b = map(int, os.environ.get("KEEP", "0:49").split(":"))
spec["outputs"] = w.spec["outputs"][a:b]
plan = rap.Plan(spec, device=0)
raw = rap.DeviceBatch(host, "cuda:0")
out = rap.DeviceOutput(plan, B, raw.sp_nnz, "cuda:0")
for _ in range(int(os.environ.get("N", "6"))):
    plan.preprocess(raw, out)
torch.cuda.synchronize()
print("ok", plan.info()["grid"])
