#!/usr/bin/env python
"""Per-CTA phase timing of one launch (rap_debug_trace; dev tool).

Stamps (%globaltimer, ns): 0 start, 1 sparse-tile queue drained, 2 dense
queue drained.
"""
import os
import sys

import numpy as np
import torch  # noqa: F401

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402

NAMES = ["start", "sparse", "dense"]


def main():
    wl = os.environ.get("WL", "c2")
    w = {"c2": synth.c2_terabyte, "c1": synth.c1_kaggle}[wl](0)
    B = int(os.environ.get("B", "65536"))
    host = synth.make_batch(w, B, seed=1)
    spec = w.spec
    keep = os.environ.get("KEEP")
    if keep:
        a, b = map(int, keep.split(":"))
        spec = dict(spec)
        spec["outputs"] = w.spec["outputs"][a:b]
    plan = rap.Plan(spec, device=0)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, B, raw.sp_nnz, "cuda:0")
    for _ in range(5):
        plan.preprocess(raw, out)
    info = plan.info()
    plan.trace_enable(4096)
    for _ in range(3):
        plan.preprocess(raw, out)
    tr = plan.trace_read(4096)[: info["grid"]].astype(np.int64)
    t0 = tr[:, 0].min()
    rel = (tr[:, :3] - t0) / 1e3
    print(f"{os.environ.get('KEEP', 'all')}: grid {info['grid']}  kernel span {rel[:, 2].max():.2f} us")
    for k in range(1, 3):
        d = rel[:, k] - rel[:, k - 1]
        print(f"  {NAMES[k - 1]:>9s}->{NAMES[k]:<9s} median {np.median(d):7.2f}  min {d.min():7.2f}  "
              f"max {d.max():7.2f}   (abs end: median {np.median(rel[:, k]):7.2f} max {rel[:, k].max():7.2f})")
    plan.close()


if __name__ == "__main__":
    main()
