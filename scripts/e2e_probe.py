#!/usr/bin/env python
"""Where the end-to-end (host-buffer) C2 step spends its time (dev tool).

Times, with CUDA events on the copy streams: the step's H2D bytes as one copy
and as the per-column copies the host entry makes, the D2H bytes, H2D and D2H
concurrently on two streams, and the pipelined `preprocess_host_async` loop
bench.py reports as e2e.  usage: e2e_probe.py [B]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_wangwdz0d24_b200 import rap, synth  # noqa: E402


def ev_time(fn, stream, reps=10):
    fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record(stream)
    for _ in range(reps):
        fn()
    e.record(stream)
    torch.cuda.synchronize()
    return s.elapsed_time(e) / reps


def main():
    B = int(sys.argv[1]) if len(sys.argv) > 1 else 65536
    dev = torch.device("cuda:0")
    w = synth.c2_terabyte(0)
    batch = synth.make_batch(w, B, seed=1000)
    plan = rap.Plan(w.spec, device=0)
    hraw = rap.DeviceBatch(batch, None, pin=True)
    hout = rap.DeviceOutput(plan, B, hraw.sp_nnz, None, pin=True)
    cols = [x for x in list(hraw.dense) + list(hraw.dense_valid) + list(hraw.sp_off) + list(hraw.sp_val) +
            list(hraw.sp_valid) if x is not None]
    h2d = sum(x.numel() * x.element_size() for x in cols)
    dcols = [torch.empty_like(x, device=dev) for x in cols]
    big_h = torch.empty(h2d, dtype=torch.uint8, pin_memory=True)
    big_d = torch.empty(h2d, dtype=torch.uint8, device=dev)
    d2h = 56_360_968
    out_h = torch.empty(d2h, dtype=torch.uint8, pin_memory=True)
    out_d = torch.empty(d2h, dtype=torch.uint8, device=dev)
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
    r = {"B": B, "h2d_bytes": h2d, "n_h2d_copies": len(cols), "d2h_bytes": d2h}

    def h2d_cols():
        with torch.cuda.stream(s1):
            for d, h in zip(dcols, cols):
                d.copy_(h, non_blocking=True)

    def h2d_one():
        with torch.cuda.stream(s1):
            big_d.copy_(big_h, non_blocking=True)

    def d2h_one():
        with torch.cuda.stream(s2):
            out_h.copy_(out_d, non_blocking=True)

    r["h2d_cols_ms"] = ev_time(h2d_cols, s1)
    r["h2d_one_ms"] = ev_time(h2d_one, s1)
    r["d2h_one_ms"] = ev_time(d2h_one, s2)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(10):
        h2d_one()
        d2h_one()
    torch.cuda.synchronize()
    r["h2d_d2h_concurrent_ms"] = (time.perf_counter() - t0) * 1e3 / 10
    # the host entries
    st = torch.cuda.current_stream(dev)
    for _ in range(3):
        plan.preprocess_host(hraw, hout, st)
    t0 = time.perf_counter()
    for _ in range(10):
        plan.preprocess_host(hraw, hout, st)
    r["preprocess_host_ms"] = (time.perf_counter() - t0) * 1e3 / 10
    t0 = time.perf_counter()
    for _ in range(10):
        plan.preprocess_host_async(hraw, hout, st)
    t1 = time.perf_counter()
    st.synchronize()
    r["preprocess_host_async_enqueue_ms"] = (t1 - t0) * 1e3 / 10
    r["preprocess_host_async_serial_ms"] = (time.perf_counter() - t0) * 1e3 / 10
    plan2 = rap.Plan(w.spec, device=0)
    hout2 = rap.DeviceOutput(plan2, B, hraw.sp_nnz, None, pin=True)
    plans, outs, streams = [plan, plan2], [hout, hout2], [s1, s2]
    for i in range(4):
        plans[i % 2].preprocess_host_async(hraw, outs[i % 2], streams[i % 2])
    torch.cuda.synchronize()
    E = 30
    t0 = time.perf_counter()
    for i in range(E):
        plans[i % 2].preprocess_host_async(hraw, outs[i % 2], streams[i % 2])
        if i >= 1:
            streams[(i - 1) % 2].synchronize()
    streams[(E - 1) % 2].synchronize()
    r["pipelined_ms"] = (time.perf_counter() - t0) * 1e3 / E
    # three plans on three streams
    plan3 = rap.Plan(w.spec, device=0)
    hout3 = rap.DeviceOutput(plan3, B, hraw.sp_nnz, None, pin=True)
    s3 = torch.cuda.Stream(dev)
    plans, outs, streams = [plan, plan2, plan3], [hout, hout2, hout3], [s1, s2, s3]
    for i in range(6):
        plans[i % 3].preprocess_host_async(hraw, outs[i % 3], streams[i % 3])
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(E):
        plans[i % 3].preprocess_host_async(hraw, outs[i % 3], streams[i % 3])
        if i >= 2:
            streams[(i - 2) % 3].synchronize()
    torch.cuda.synchronize()
    r["pipelined3_ms"] = (time.perf_counter() - t0) * 1e3 / E
    # copies alone, the same pipeline shape: per-column H2D on one stream,
    # one D2H on the other, alternating
    outs_h = [out_h, torch.empty_like(out_h, pin_memory=True)]
    ss = [s1, s2]

    def step(i):
        with torch.cuda.stream(ss[i % 2]):
            for d, h in zip(dcols, cols):
                d.copy_(h, non_blocking=True)
            outs_h[i % 2].copy_(out_d, non_blocking=True)

    for i in range(4):
        step(i)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(E):
        step(i)
        if i >= 1:
            ss[(i - 1) % 2].synchronize()
    torch.cuda.synchronize()
    r["copies_only_pipelined_ms"] = (time.perf_counter() - t0) * 1e3 / E
    print(json.dumps(r))


if __name__ == "__main__":
    main()
