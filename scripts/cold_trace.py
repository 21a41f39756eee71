#!/usr/bin/env python
"""Warm vs cold (rotating input/output sets, as bench.py times) kernel time of
one workload, plus per-CTA phase stamps of a cold launch (dev tool).

WL=c2|c1|c4, B=rows, NSETS=rotating sets (default 6), KMODE=rap kernel mode."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402

NAMES = ["start", "published", "dense", "seen", "bases", "ids"]


def timed(plan, sets, n, stream):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
    for i in range(n):
        r, o = sets[i % len(sets)]
        ev[i][0].record(stream)
        plan.preprocess(r, o, stream)
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    return float(np.median([a.elapsed_time(b) for a, b in ev])) * 1e3


def graph_time(plan, sets, reps, stream):
    """Per-launch time of 2 x len(sets) launches captured in one CUDA graph (no host gaps)."""
    g = torch.cuda.CUDAGraph()
    s2 = torch.cuda.Stream()
    s2.wait_stream(stream)
    with torch.cuda.stream(s2):
        with torch.cuda.graph(g, stream=s2):
            for i in range(2 * len(sets)):
                r, o = sets[i % len(sets)]
                plan.preprocess(r, o, s2)
    torch.cuda.synchronize()
    g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for _ in range(reps):
        g.replay()
    b.record(stream)
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1e3 / (reps * 2 * len(sets))


def stamps(plan, sets, stream, label):
    plan.trace_enable(4096)
    for i in range(len(sets) + 1):
        r, o = sets[i % len(sets)]
        plan.preprocess(r, o, stream)
    torch.cuda.synchronize()
    info = plan.info()
    tr = plan.trace_read(4096)[: info["grid"]].astype(np.int64)
    plan.trace_disable()
    ok = (tr[:, 0] > 0) & (tr[:, 5] > 0)
    tr = tr[ok]
    t0 = tr[:, 0].min()
    rel = (tr[:, :6] - t0) / 1e3
    print(f"  [{label}] span {rel[:, 5].max():.2f} us over {len(tr)} CTAs")
    for k in range(1, 6):
        d = rel[:, k] - rel[:, k - 1]
        print(f"    {NAMES[k - 1]:>9s}->{NAMES[k]:<9s} median {np.median(d):7.2f} max {d.max():7.2f}  "
              f"(abs end median {np.median(rel[:, k]):7.2f} max {rel[:, k].max():7.2f})")
    ex = (tr[:, 6:16] - t0) / 1e3
    for k, nm in enumerate(["slots ready", "setup done", "chunk0 staged", "first dense", "base loads",
                            "base sync", "base sums", "totals stored", "kernel end", "dense warp end"]):
        v = ex[:, k]
        v = v[v > -1e6]
        if len(v):
            print(f"    {nm:>14s}: median abs {np.median(v):7.2f} max {v.max():7.2f}")


def main():
    wl = os.environ.get("WL", "c2")
    w = {"c2": synth.c2_terabyte, "c1": synth.c1_kaggle, "c4": synth.c4_multihot}[wl](0)
    B = int(os.environ.get("B", "65536"))
    nsets = int(os.environ.get("NSETS", "6"))
    plan = rap.Plan(w.spec, device=0)
    if os.environ.get("KMODE"):
        plan.set_kernel(int(os.environ["KMODE"]))
    sets = []
    for i in range(nsets):
        h = synth.make_batch(w, B, seed=1000 + 97 * i)
        r = rap.DeviceBatch(h, "cuda:0")
        sets.append((r, rap.DeviceOutput(plan, B, r.sp_nnz, "cuda:0")))
    stream = torch.cuda.current_stream()
    timed(plan, sets, 20, stream)
    info = plan.info()
    tag = os.environ.get("TAG", "")
    warm = timed(plan, sets[:1], 200, stream)
    x = torch.zeros(1, device="cuda:0")
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(100)]
    for a, b in ev:
        a.record(stream)
        x.add_(1)
        b.record(stream)
    torch.cuda.synchronize()
    print(f"  empty-ish kernel (1-elem add) event time {np.median([a.elapsed_time(b) for a, b in ev]) * 1e3:.2f} us")
    cold = timed(plan, sets, 300, stream)
    mx = np.max([np.asarray(r.sp_nnz) for r, _ in sets], axis=0)
    bigs = [rap.DeviceOutput(plan, B, mx, "cuda:0") for _ in sets]
    ins = [(r, bigs[0]) for r, _ in sets]   # inputs rotate, one output set
    outs = [(sets[0][0], o) for o in bigs]  # one input set, outputs rotate
    cold_in = timed(plan, ins, 300, stream)
    cold_out = timed(plan, outs, 300, stream)
    print(f"  inputs cold only {cold_in:.2f} us, outputs cold only {cold_out:.2f} us")
    gw = graph_time(plan, sets[:1], 50, stream)
    gc = graph_time(plan, sets, 50, stream)
    print(f"  graph replay per launch: warm {gw:.2f} us, cold {gc:.2f} us")
    print(f"{wl} B={B} {tag}: kernel {info.get('kernel_last')} grid {info['grid']} rows {info.get('rb_rows')} "
          f"groups {info.get('rb_feature_groups')} jit ctas/sm {info.get('jit_ctas_per_sm')} "
          f"smem {info.get('rows_smem_bytes')}: warm {warm:.2f} us, cold ({nsets} sets) {cold:.2f} us")
    if os.environ.get("STAMPS", "1") == "1":
        stamps(plan, sets[:1], stream, "warm")
        stamps(plan, sets, stream, "cold")
    plan.close()


if __name__ == "__main__":
    main()
