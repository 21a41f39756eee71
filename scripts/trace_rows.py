#!/usr/bin/env python
"""Per-CTA phase timing of one row-block launch (rap_debug_trace; dev tool).

Stamps (%globaltimer, ns) of rap_rows.cu: 0 start, 1 totals published,
2 dense blocks done, 3 all words seen, 4 bases reduced, 5 ids written;
6-13 finer points of the row-block skeleton (rap_rows_skel.cuh)."""
import os
import sys

import numpy as np
import torch  # noqa: F401

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402

NAMES = ["start", "published", "dense", "seen", "bases", "ids"]


def main():
    wl = os.environ.get("WL", "c2")
    w = {"c2": synth.c2_terabyte, "c1": synth.c1_kaggle, "c4": synth.c4_multihot}[wl](0)
    B = int(os.environ.get("B", "65536"))
    host = synth.make_batch(w, B, seed=1)
    plan = rap.Plan(w.spec, device=0)
    plan.set_kernel(int(os.environ.get("KMODE", rap.KERNEL_ROWS)))
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, B, raw.sp_nnz, "cuda:0")
    for _ in range(5):
        plan.preprocess(raw, out)
    plan.trace_enable(4096)
    for _ in range(3):
        plan.preprocess(raw, out)
    info = plan.info()
    grid = info["grid"]
    tr = plan.trace_read(4096)[:grid].astype(np.int64)
    ok = (tr[:, 0] > 0) & (tr[:, 5] > 0)
    tr = tr[ok]
    t0 = tr[:, 0].min()
    rel = (tr[:, :6] - t0) / 1e3
    print(f"{wl} B={B}: grid {grid} ({info['rb_row_blocks']} row blocks x {info['rb_feature_groups']} groups, "
          f"{info['rb_rows']} rows), {info['rows_ctas_per_sm']} CTAs/SM, smem {info['rows_smem_bytes']}, "
          f"memo {info['rb_memo_slots']}; span {rel[:, 5].max():.2f} us over {len(tr)} CTAs")
    for k in range(1, 6):
        d = rel[:, k] - rel[:, k - 1]
        print(f"  {NAMES[k - 1]:>9s}->{NAMES[k]:<9s} median {np.median(d):7.2f}  max {d.max():7.2f}   "
              f"(abs end median {np.median(rel[:, k]):7.2f} max {rel[:, k].max():7.2f})")
    print(f"  CTA start: p50 {np.percentile(rel[:, 0], 50):.2f} p90 {np.percentile(rel[:, 0], 90):.2f} "
          f"max {rel[:, 0].max():.2f} us")
    ex = (tr[:, 6:14] - t0) / 1e3
    for k, nm in enumerate(["slots ready", "setup done", "chunk0 staged", "first dense block", "base loads+redux",
                            "base sync", "base sums", "totals stored"]):
        v = ex[:, k]
        v = v[v > -1e6]
        if len(v):
            print(f"  {nm:>18s}: median abs {np.median(v):7.2f} us  max {v.max():7.2f}")
    plan.close()


if __name__ == "__main__":
    main()
