#!/usr/bin/env python
"""Latency floor probes (dev tool): one-feature graphs at tiny and full batch."""
import copy, os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402
from scripts.probe import time_spec, subspec  # noqa: E402

w = synth.c2_terabyte(0)
outs = w.spec["outputs"]
for B in (128, 4096, 65536):
    host = synth.make_batch(w, B, seed=1)
    for name, keep in [("1 sparse", outs[15:16]), ("1 ngram", outs[41:42]), ("1 dense", outs[:1]), ("full", outs)]:
        for budget in (0, 1):
            us, info = time_spec(subspec(w.spec, keep), host, steps=100, budget=budget)
            print(f"B={B:6d} {name:10s} budget={budget} {us:8.2f} us grid {info['grid']}", flush=True)
