#!/usr/bin/env python
"""Per-CTA phase timing of one launch (rap_debug_trace; dev tool).

Stamps (%globaltimer, ns): 0 start, 1 length pass published, 2 dense blocks
done, 3 predecessors' aggregates read, 4 sparse tiles written.
"""
import os
import sys

import numpy as np
import torch  # noqa: F401

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402

NAMES = ["start", "lengths", "dense", "wait", "values"]


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
    rel = (tr[:, :5] - t0) / 1e3
    rel[:, 3] = np.maximum(rel[:, 3], rel[:, 2])
    print(f"{os.environ.get('KEEP', 'all')}: grid {info['grid']}  kernel span {rel[:, 4].max():.2f} us")
    for k in range(1, 5):
        d = rel[:, k] - rel[:, k - 1]
        print(f"  {NAMES[k - 1]:>9s}->{NAMES[k]:<9s} median {np.median(d):7.2f}  min {d.min():7.2f}  "
              f"max {d.max():7.2f}   (abs end: median {np.median(rel[:, k]):7.2f} max {rel[:, k].max():7.2f})")
    st = rel[:, 0]
    print(f"  CTA start offsets: p50 {np.percentile(st, 50):.2f} p90 {np.percentile(st, 90):.2f} max {st.max():.2f} us;"
          f" distinct SMs {len(set(tr[:, 6].tolist()))}")
    order = np.argsort(-rel[:, 4])[:6]
    for i in order:
        print(f"  slowest CTA blk {i} rank {tr[i, 7]} sm {tr[i, 6]}: " + " ".join(f"{x:7.2f}" for x in rel[i, :5]))
    T = (B + 127) // 128
    s0 = tr[:, 5] & 0xffffffff
    ns = tr[:, 5] >> 32
    vt = rel[:, 4] - rel[:, 3]
    feats = {}
    for i in range(len(tr)):
        if ns[i] > 0:
            feats.setdefault(int(s0[i] // T), []).append((vt[i], ns[i]))
    print("  per first-feature: feature: n_ctas, median values-phase us, median tiles")
    print("   " + "  ".join(f"{f}:{len(v)},{np.median([a for a, _ in v]):.0f},{np.median([b for _, b in v]):.0f}"
                          for f, v in sorted(feats.items())))
    cl = tr[:, 8:13].astype(np.int64)
    okc = (cl > 0).all(axis=1)
    if okc.any():
        d = np.diff(cl[okc], axis=1)
        print("  first canon chunk of warp 0 (cycles, median over CTAs): stage offsets %d  ids %d  canon %d  stores %d" %
              tuple(np.median(d, axis=0)))
    cl = tr[:, 13:16].astype(np.int64)
    okc = (cl > 0).all(axis=1)
    if okc.any():
        d = np.diff(cl[okc], axis=1)
        print("  first fast-ngram tile of warp 0 (cycles, median): params+quads+values %d  hash+stores %d" %
              tuple(np.median(d, axis=0)))
    cl = tr[:, 16:21].astype(np.int64)
    okc = (cl > 0).all(axis=1)
    if okc.any():
        d = np.diff(cl[okc], axis=1)
        print("  first dense block (cycles, median): prog+issue %d  staged wait %d  compute %d  store %d" %
              tuple(np.median(d, axis=0)))
    cl = tr[:, 21:24].astype(np.int64)
    okc = (cl > 0).all(axis=1)
    if okc.any():
        d = np.diff(cl[okc], axis=1)
        print("  phase L (cycles, median): warp 0 loop %d  block wait %d   (p90 %d %d)" %
              (tuple(np.median(d, axis=0)) + tuple(np.percentile(d, 90, axis=0))))
    plan.close()


if __name__ == "__main__":
    main()
