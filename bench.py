#!/usr/bin/env python
"""Benchmark of the fused RAP preprocessing kernel (BASELINE.json metric:
preprocessed samples/s, % of HBM roofline).

A step = one rap_preprocess launch over one synthetic Criteo-Terabyte-shaped
batch (config 2, 65536 rows, the full 152-op graph) — every §8(a) row of the
hot path.  Inputs are resident in HBM when the timed region starts; the
batch/output sets are rotated so their total exceeds 2x the L2 (126 MB).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl rap|reference]

Prints ONE JSON line on rank 0.  `--impl reference` times the CPU oracle (the
task's reference arm for a paper-only reference) on bounded samples.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "preprocessed samples/s"
UNIT = "samples/s"
WORKLOADS = {"c2": ("criteo_terabyte_c2", 65536), "c1": ("criteo_kaggle_c1", 4096), "c4": ("multihot_c4", 131072),
             "plan2": ("table3_plan2", 65536), "plan3": ("table3_plan3", 65536)}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3000)
    ap.add_argument("--warmup", type=int, default=50)
    ap.add_argument("--impl", default="rap", choices=["rap", "reference"])
    ap.add_argument("--workload", default="c2", choices=list(WORKLOADS))
    ap.add_argument("--batch", type=int, default=0, help="override rows per batch")
    ap.add_argument("--budget", type=int, default=0, help="SM budget (0 = all SMs)")
    ap.add_argument("--e2e-steps", type=int, default=30)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no clocks / e2e / cpu)")
    ap.add_argument("--no-corun", action="store_true", help="skip the co-run training-slowdown measurement")
    ap.add_argument("--no-fusion", action="store_true", help="skip the one-launch-per-feature fusion ablation")
    ap.add_argument("--corun-budgets", default="16,37,74,148", help="SM budgets of the co-run sweep")
    ap.add_argument("--placement", default="balanced", choices=["balanced", "round_robin", "skewed"],
                    help="N>1: table placement (DESIGN.md §10)")
    ap.add_argument("--imbalance-tol", type=float, default=0.10, help="N>1: residual move threshold")
    ap.add_argument("--no-c4", action="store_true", help="skip the config-4 (multi-hot) sub-measurement")
    ap.add_argument("--c4-batch", type=int, default=16384, help="rows of the config-4 sub-measurement")
    ap.add_argument("--no-plans", action="store_true", help="skip the Table 3 Plan 2 / 3 sub-measurements")
    ap.add_argument("--ngram-sweep", default="", help="e.g. 8,16,32,64: growing-NGram co-run sweep (Fig 11 analog)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="N>1: gloo = host-staged exchange (ranks sharing one GPU: tests)")
    return ap.parse_args()


def workload(name, seed=0):
    from paper_conf_asplos_wangwdz0d24_b200 import synth

    if name == "c2":
        return synth.c2_terabyte(seed)
    if name == "c1":
        return synth.c1_kaggle(seed)
    if name in ("plan2", "plan3"):
        return synth.plan_graph(int(name[-1]), seed)
    return synth.c4_multihot(seed)


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """Samples SM clock and throttle reasons with NVML while the timed region runs."""

    REASONS = {"hw_slowdown": 0x8, "hw_thermal_slowdown": 0x40, "sw_thermal_slowdown": 0x20,
               "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, index):
        self.samples, self.reasons = [], set()
        self.ok = False
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # noqa: BLE001
            self.err = str(e)
        self._stop = threading.Event()

    def _run(self):
        while not self._stop.is_set():
            self.sample()
            time.sleep(0.002)

    def sample(self):
        try:
            mhz = self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM)
            r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            self.samples.append(mhz)
            for k, bit in self.REASONS.items():
                if r & bit:
                    self.reasons.add(k)
        except Exception:  # noqa: BLE001
            pass

    def __enter__(self):
        if self.ok:
            self.sample()
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()
            self.sample()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ----------------------------------------------------------------------------- helpers
def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:  # noqa: BLE001
        return 6650.0, "fallback"


def traffic_from_profile(workload_name):
    """DRAM bytes per launch from the committed ncu --set full summary, if any."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(workload_name)
    except Exception:  # noqa: BLE001
        return None


def issue_roofline(workload_name, kern_ms):
    """The instruction-issue roofline of the same kernel from the committed ncu
    capture (profiles/issue.json): its warp instructions at one issue per
    SMSP per cycle (148 SMs x 4 SMSPs at the max SM clock) against the
    measured time -- the limiter when the HBM fraction is low."""
    p = os.path.join(ROOT, "profiles", "issue.json")
    try:
        with open(p) as f:
            d = json.load(f)[workload_name]
    except Exception:  # noqa: BLE001
        return None
    ideal_ms = d["warp_inst_per_launch"] / (148 * 4 * 1.965e9) * 1e3
    return {"warp_inst_per_launch": d["warp_inst_per_launch"], "ideal_issue_ms": ideal_ms,
            "frac": ideal_ms / kern_ms, "ncu_issue_active_pct": d["issue_active_pct"],
            "ncu_warps_active_pct": d["warps_active_pct"], "source": d.get("summary"),
            "limiter": "latency: few resident warps, dependent id-load -> probe -> hash -> store chains"}


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_baseline(w, seconds, rows=8192):
    """The oracle, as it stands, on a bounded sample of the same workload:
    single-threaded, and on every core the process may use (one row slice per
    thread; ctypes releases the GIL inside the C oracle)."""
    from concurrent.futures import ThreadPoolExecutor

    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import synth

    host = synth.make_batch(w, rows, seed=101)
    oracle.lib()
    n = 0
    t0 = time.perf_counter()
    while True:
        r = oracle.run(w.spec, host)
        assert r["status"] == "OK"
        n += 1
        if time.perf_counter() - t0 >= seconds / 2:
            break
    dt1 = time.perf_counter() - t0
    one = n * rows / dt1
    cores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
    per = max(256, rows // 4)
    slices = [synth.make_batch(w, per, seed=300 + i) for i in range(cores)]
    done = [0] * cores

    def work(i):
        t = time.perf_counter()
        while time.perf_counter() - t < seconds / 2:
            assert oracle.run(w.spec, slices[i])["status"] == "OK"
            done[i] += 1

    t0 = time.perf_counter()
    with ThreadPoolExecutor(cores) as ex:
        list(ex.map(work, range(cores)))
    dtm = time.perf_counter() - t0
    allc = sum(done) * per / dtm
    return {"value": allc, "unit": UNIT, "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
            "value_1thread": one,
            "sample": f"{w.name}: {n} x {rows}-row batches on 1 thread ({dt1:.1f} s), then {sum(done)} x {per}-row "
                      f"slices over {cores} threads ({dtm:.1f} s); plain C oracle, untuned"}


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


# ----------------------------------------------------------------------------- reference arm
def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import synth

    wname, B = WORKLOADS[args.workload]
    B = args.batch or B
    w = workload(args.workload)
    oracle.lib()
    total_steps = args.steps + args.warmup
    budget_s = 90.0
    # oracle throughput ~6e4 rows/s on C2: size each step so the run stays within ~budget_s
    rows = int(max(32, min(B, 6e4 * budget_s / max(total_steps, 1))))
    host = synth.make_batch(w, rows, seed=202)
    for _ in range(args.warmup):
        oracle.run(w.spec, host)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        r = oracle.run(w.spec, host)
    dt = time.perf_counter() - t0
    assert r["status"] == "OK"
    value = args.steps * rows / dt
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 0,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int64+f32",
            "data": "synthetic",
            "config": {"workload": wname, "batch": B, "sample_rows_per_step": rows, "parallelism": "cpu-1thread"},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"{rows}-row sample of {wname} per step (seed 202), single-threaded C oracle"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------------------------- GPU arm
def run_rap(args):
    import torch

    rank, world, local = dist_env()
    if world > 1:
        return run_sharded(args)
    torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth

    wname, B = WORKLOADS[args.workload]
    B = args.batch or B
    w = workload(args.workload)
    # Replicas: with N > 1 every rank preprocesses its own batch of B rows (data-parallel
    # batches, no data-path collective) -> weak scaling, value = all ranks' rows / max time.
    plan = rap.Plan(w.spec, device=dev.index, sm_budget=args.budget)
    props = torch.cuda.get_device_properties(dev)
    l2 = getattr(props, "L2_cache_size", 126 * 2**20)

    first = synth.make_batch(w, B, seed=1000 + rank)
    raw0 = rap.DeviceBatch(first, dev)
    out0 = rap.DeviceOutput(plan, B, raw0.sp_nnz, dev)
    d_out, f_out, vb = out0.d_out, out0.f_out, out0.bound
    # algorithmic bytes of one launch: measured from the produced output
    plan.preprocess(raw0, out0)
    torch.cuda.synchronize()
    n_vals = int(out0.offsets[-1].item())
    alg_bytes = synth.algorithmic_bytes(w.spec, first, n_vals)
    set_bytes = alg_bytes
    nsets = 1 if args.profile else max(4, math.ceil(3 * l2 / max(set_bytes, 1)))
    sets = [(raw0, out0)]
    for i in range(1, nsets):
        h = synth.make_batch(w, B, seed=1000 + rank + 97 * i)
        r = rap.DeviceBatch(h, dev)
        sets.append((r, rap.DeviceOutput(plan, B, r.sp_nnz, dev)))
    stream = torch.cuda.current_stream(dev)

    for i in range(args.warmup):
        r, o = sets[i % nsets]
        plan.preprocess(r, o, stream)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()

    K = args.steps
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(dev.index) if not args.profile else None
    ctx = sampler if sampler else _Null()
    # The timed steps are replays of CUDA graphs holding the rap_preprocess
    # launches (one per rotating input/output set, back to back on the
    # stream), so the per-call host cost (ctypes, C-ABI validation) does not
    # leave the GPU idle between launches; exactly K launches are timed.
    graphs = step_graphs(plan, sets, K, stream) if not args.profile and world == 1 else None
    with ctx:
        t_start.record(stream)
        if graphs is not None:
            g_full, reps, g_rem = graphs
            for _ in range(reps):
                g_full.replay()
            if g_rem is not None:
                g_rem.replay()
        else:
            for i in range(K):
                r, o = sets[i % nsets]
                plan.preprocess(r, o, stream)
        t_end.record(stream)
        t_end.synchronize()
    torch.cuda.synchronize()
    info = plan.info()  # the launches just timed (kernel, grid)
    total_ms = t_start.elapsed_time(t_end)
    # average launch duration of the kernel inside the timed region: the graphs
    # hold only its launches, so the region's time over K launches (inter-kernel
    # gaps included, a conservative bound)
    kern_ms = total_ms / K
    # per-call launches bracketed by events, for reference (not the timed region)
    eager = None
    if not args.profile:
        KE = min(K, 300)
        ev_s = [torch.cuda.Event(enable_timing=True) for _ in range(KE)]
        ev_e = [torch.cuda.Event(enable_timing=True) for _ in range(KE)]
        for i in range(KE):
            r, o = sets[i % nsets]
            ev_s[i].record(stream)
            plan.preprocess(r, o, stream)
            ev_e[i].record(stream)
        torch.cuda.synchronize()
        eager = {"kernel_ms": float(np.mean([ev_s[i].elapsed_time(ev_e[i]) for i in range(KE)])), "launches": KE,
                 "what": "one rap_preprocess call per step from Python, each bracketed by CUDA events"}
    if world > 1:
        import torch.distributed as dist

        t = torch.tensor([total_ms, kern_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms, kern_ms = float(t[0]), float(t[1])
        dist.barrier()
    ms_per_step = total_ms / K
    value = world * B * K / (total_ms / 1e3)

    # ---- correctness spot check of the last launch (cheap invariants, not the oracle)
    o = sets[(K - 1) % nsets][1]
    offs = o.offsets
    assert int(offs[0]) == 0 and bool((offs[1:] >= offs[:-1]).all())

    # ---- end to end through the C ABI with host buffers
    e2e = None
    if not args.no_e2e and not args.profile:
        hraw = rap.DeviceBatch(first, None, pin=True)
        hout = rap.DeviceOutput(plan, B, hraw.sp_nnz, None, pin=True)
        h2d = sum(x.numel() * x.element_size() for x in hraw.dense)
        h2d += sum(x.numel() * x.element_size() for x in hraw.dense_valid if x is not None)
        h2d += sum(x.numel() * x.element_size() for x in hraw.sp_off)
        h2d += sum(int(n) * 8 for n in hraw.sp_nnz)
        h2d += sum(x.numel() * x.element_size() for x in hraw.sp_valid if x is not None)
        # values: exactly offsets[end] ids (the pinned-output copy kernel, include/rap.h)
        d2h = (B * d_out * 4) + (B * f_out * 4) + (B * f_out + 1) * 8 + n_vals * 8
        for _ in range(3):
            plan.preprocess_host(hraw, hout, stream)
        if world > 1:
            torch.distributed.barrier()
        E = max(3, args.e2e_steps)
        t0 = time.perf_counter()
        for _ in range(E):
            plan.preprocess_host(hraw, hout, stream)
        dt_sync = time.perf_counter() - t0
        # pipelined: two plans on two streams (rap_preprocess_host_async), so
        # batch i+1's H2D copies and kernel overlap batch i's D2H copies; each
        # step still copies its inputs in and its outputs out
        # three plans deep: batch i+2's inputs cross while i+1 runs and i's
        # outputs come back (scripts/e2e_probe.py: 2 deep 1.38 ms, 3 deep 1.31)
        NP = 3
        extra = [rap.Plan(w.spec, device=dev.index, sm_budget=args.budget) for _ in range(NP - 1)]
        plans = [plan] + extra
        outs = [hout] + [rap.DeviceOutput(p, B, hraw.sp_nnz, None, pin=True) for p in extra]
        streams = [torch.cuda.Stream(dev) for _ in range(NP)]
        for i in range(2 * NP):
            plans[i % NP].preprocess_host_async(hraw, outs[i % NP], streams[i % NP])
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for i in range(E):
            plans[i % NP].preprocess_host_async(hraw, outs[i % NP], streams[i % NP])
            if i >= NP - 1:
                streams[(i - NP + 1) % NP].synchronize()  # batch i-NP+1's outputs are in host memory
        for st_ in streams:
            st_.synchronize()
        dt = time.perf_counter() - t0
        for p in extra:
            p.close()
        if world > 1:
            import torch.distributed as dist

            t = torch.tensor([dt], device=dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dt = float(t[0])
        e2e = {"value": world * B * E / dt, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h), "steps": E,
               "mode": "rap_preprocess_host_async, 3 plans x 3 streams (H2D gather / kernel of i+1, i+2 overlap D2H of i)",
               "value_synchronous": world * B * E / dt_sync}

    peak, peak_kind = measured_peaks()
    achieved = alg_bytes / (kern_ms / 1e3) / 1e9
    traffic = traffic_from_profile(wname)
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": traffic, "peak_source": peak_kind, "alg_bytes_per_launch": int(alg_bytes),
            "kernel_ms": kern_ms, "eager": eager,
            "traffic_note": "dram read+write of the committed ncu --set full capture (profiles/traffic.json); "
                            "output lines still dirty in the 126 MB L2 at kernel end are not counted",
            "issue": issue_roofline(wname, kern_ms)}
    clocks = sampler.summary() if sampler else None
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and not args.profile:
        cpu = cpu_baseline(w, args.cpu_seconds)
    graph = None
    if world == 1 and not args.profile and args.workload in ("c1", "c2"):
        try:
            graph = graph_replay(plan, sets, B, dev, steps=K, alg_bytes=alg_bytes)
        except Exception as ex:  # reported, never silently replaced
            graph = {"error": repr(ex)[:300]}
            torch.cuda.synchronize()
    fusion = None
    if world == 1 and not args.no_fusion and not args.profile and args.workload in ("c1", "c2"):
        fusion = fusion_ablation(w, sets, B, dev, stream, kern_ms, steps=min(K, 200))
        fusion["perop"] = perop_baseline(w, first, dev, kern_ms)
    corun = None
    if world == 1 and not args.no_corun and not args.profile and args.workload == "c2":
        from paper_conf_asplos_wangwdz0d24_b200 import corun as cr

        train = cr.DLRMStep(dev)
        budgets = [int(b) for b in args.corun_budgets.split(",") if b]
        corun = cr.measure(plan, sets, train, budgets, choose=(B, sets[0][0].sp_nnz), partitions=(8, 16, 40))
        corun["training"] = "synthetic DLRM step (DESIGN.md §12): 26 tables x 128 fp32 (TB share at 8 GPUs), batch 8192"
        # layer-aligned scheduling (Algorithm 1): chunks launched as their layers begin
        layer_us = train.layer_times_us()
        corun["layer_aligned"] = {"layer_us": layer_us, "per_budget": []}
        lsets = [r for r, _ in sets[:2]]
        for lb in (0, 8, 2):
            lap = cr.LayerAlignedPrep(w.spec, B, sets[0][0].sp_nnz, layer_us, device=dev.index, budget=lb)
            louts = [lap.output(r.sp_nnz, dev) for r in lsets]
            t_l, p_l, a_l = cr.measure_layer_aligned(lap, lsets, louts, train)
            corun["layer_aligned"]["per_budget"].append(
                {"pack_budget": lb, "chunks": lap.describe(), "train_step_alone_ms": a_l, "train_step_corun_ms": t_l,
                 "prep_done_ms": p_l, "slowdown": t_l / a_l - 1.0, "prep_hidden": p_l <= t_l})
            lap.close()
            del louts
        del train
        torch.cuda.empty_cache()
    ngram_sweep = None
    if world == 1 and not args.profile and args.ngram_sweep:
        ngram_sweep = ngram_sweep_point(dev, B, [int(k) for k in args.ngram_sweep.split(",") if k])
    mapping = None
    if world == 1 and not args.profile and args.workload in ("c1", "c2"):
        mapping = mapping_point(plan, w.spec, raw0.sp_nnz, B, kern_ms)
    c4 = None
    if world == 1 and not args.profile and not args.no_c4 and args.workload != "c4":
        c4 = c4_point(dev, args.c4_batch, steps=20)
    plans = None
    if world == 1 and not args.profile and not args.no_plans and args.workload in ("c1", "c2"):
        plans = [plan_point(dev, p, 65536) for p in (2, 3)]
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": args.warmup,
                "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
                "dtype": "int64+f32", "data": "synthetic",
                "config": {"workload": wname, "batch": B, "graph_ops": len(w.spec["nodes"]),
                           "dense_out_cols": d_out, "sparse_out_features": f_out,
                           "parallelism": "replicas" if world > 1 else "single-gpu",
                           "sm_budget": info["sm_budget"], "grid": info["grid"],
                           "kernel": KERNEL_NAMES.get(info["kernel_last"], str(info["kernel_last"])),
                           "jit_compile_s": round(info["jit_compile_seconds"], 2),
                           "l2_policy": f"rotate {nsets} distinct input/output sets, {nsets * set_bytes / 2**20:.0f} MB "
                                        f"total vs L2 {l2 / 2**20:.0f} MB"},
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks, "gpu_launches": K,
                "corun": corun, "fusion": fusion, "graph": graph, "c4": c4, "plans": plans, "mapping": mapping,
                "ngram_sweep": ngram_sweep}
        print(json.dumps(line), flush=True)
    plan.close()
    if world > 1:
        import torch.distributed as dist

        dist.destroy_process_group()
    return 0


KERNEL_NAMES = {1: "tiled", 2: "rows (interpreted)", 3: "rows (generated, NVRTC sm_100a)"}


def ngram_sweep_point(dev, B, counts):
    """Fig 11 analog: the C2 graph with a growing number
    of trigram features beside the fixed synthetic DLRM training step: per
    count, the fused launch alone and the training step's slowdown when the
    launch co-runs on a low-priority stream at the full budget and at the
    budget rap_choose_budget picks (the paper's turning point: a > 10 % rise)."""
    import torch

    from paper_conf_asplos_wangwdz0d24_b200 import corun as cr, rap, synth

    train = cr.DLRMStep(dev)
    out = []
    for k in counts:
        w = synth.c2_terabyte(0, n_ngram=k)
        plan = rap.Plan(w.spec, device=dev.index)
        sets = []
        for i in range(2):
            h = synth.make_batch(w, B, seed=300 + i)
            r = rap.DeviceBatch(h, dev)
            sets.append((r, rap.DeviceOutput(plan, B, r.sp_nnz, dev)))
        m = cr.measure(plan, sets, train, [plan.info()["sm_budget"]], steps=12, warmup=3,
                       choose=(B, sets[0][0].sp_nnz))
        full = m["per_budget"][0]
        out.append({"n_ngram": k, "sparse_outputs": 26 + k, "kernel": KERNEL_NAMES.get(plan.info()["kernel_last"], "?"),
                    "prep_alone_ms": full["prep_alone_ms"], "slowdown_full_budget": full["slowdown"],
                    "chosen_budget": m["chosen"]["sm_budget"], "slowdown_chosen": m["chosen"]["slowdown"],
                    "train_step_alone_ms": m["train_step_alone_ms"]})
        plan.close()
        del sets
        torch.cuda.empty_cache()
    del train
    return out


def mapping_point(plan, spec, sp_nnz, B, kern_ms, world=8, B_eval=None):
    """Fig 12 analog (§7.2), model-based: the
    C2 graph's outputs on `world` ranks with a skewed consumer placement (rank
    0 consumes ~2x the mean, rap_place "skewed"), the per-rank preprocessing
    time of three mappings under the plan's cost model scaled to this GPU's
    measured C2 kernel time and a 700 GB/s, 20 us link: data locality (every
    graph on its consumer), data parallel (every rank the whole graph on its
    batch shard, outputs all-to-all), and the joint mapping loop
    (rap_place_joint).  One GPU here: no multi-GPU run behind these numbers."""
    from paper_conf_asplos_wangwdz0d24_b200 import dist

    import numpy as np

    u = kern_ms * 1e3 / max(float(sum(plan.output_costs(B, sp_nnz))), 1e-9)  # this GPU's scale
    if B_eval and B_eval != B:  # the config's own batch (ids scale with rows)
        sp_nnz = (np.asarray(sp_nnz, dtype=np.float64) * (B_eval / B)).astype(np.int64)
        B = B_eval
    costs = plan.output_costs(B, sp_nnz)
    cm = dist.CommModel(us_per_unit=u)
    col = dist.colocation(spec)
    rb = dist.row_bytes(spec, sp_nnz, B)
    home = dist.place(costs, col, world, "skewed", B, None).owner
    joint = dist.place_joint(costs, col, home, world, B, cm, rb, 0.0)
    dl = dist.place_joint(costs, col, home, world, B, dist.CommModel(u, 1e-9, 1e12), rb, 0.0)  # no move pays
    comp = float(sum(costs)) * u / world
    xfer = cm.link_latency_us + sum(rb) * (B / world) * (world - 1) / world / (1e3 * cm.link_gbs)
    return {"what": f"model-based per-rank preprocessing time (us), {len(costs)} outputs, B = {B}, {world} ranks, "
                    "skewed consumers",
            "us_per_cost_unit": u, "link_gbs": cm.link_gbs, "link_latency_us": cm.link_latency_us,
            "data_locality": {"max_us": max(dl.times), "times_us": dl.times},
            "data_parallel": {"max_us": comp + xfer, "compute_us": comp, "all_to_all_us": xfer},
            "joint": {"max_us": max(joint.times), "times_us": joint.times, "moves": joint.moves},
            "dl_over_joint": max(dl.times) / max(max(joint.times), 1e-9),
            "dp_over_joint": (comp + xfer) / max(max(joint.times), 1e-9)}


def c4_point(dev, B, steps=20):
    """Config 4 (512 multi-hot features, mean 20 ids, FirstX(32)) at B rows on
    this GPU: kernel time and HBM fraction of the launch (the tiled kernel's
    element-parallel multi-id tiles).  Rotating 2 batches (each > the L2)."""
    import torch

    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth

    w = synth.c4_multihot(0)
    plan = rap.Plan(w.spec, device=dev.index)
    sets = []
    for i in range(2):
        h = synth.make_batch(w, B, seed=700 + i)
        r = rap.DeviceBatch(h, dev)
        sets.append((h, r, rap.DeviceOutput(plan, B, r.sp_nnz, dev)))
    stream = torch.cuda.current_stream(dev)
    for i in range(4):
        plan.preprocess(sets[i % 2][1], sets[i % 2][2], stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for i in range(steps):
        plan.preprocess(sets[i % 2][1], sets[i % 2][2], stream)
    e1.record(stream)
    e1.synchronize()
    ms = e0.elapsed_time(e1) / steps
    n_vals = int(sets[(steps - 1) % 2][2].offsets[-1].item())
    alg = synth.algorithmic_bytes(w.spec, sets[(steps - 1) % 2][0], n_vals)
    peak, _ = measured_peaks()
    info = plan.info()
    # config 4's 8-GPU mapping (its full 131072-row batch), model-based
    mapping = mapping_point(plan, w.spec, sets[0][1].sp_nnz, B, ms, world=8, B_eval=131072)
    plan.close()
    del sets
    torch.cuda.empty_cache()
    gbs = alg / (ms / 1e3) / 1e9
    return {"workload": "multihot_c4", "batch": B, "kernel_ms": ms, "value": B / (ms / 1e3), "unit": UNIT,
            "alg_bytes_per_launch": int(alg), "achieved_gbs": gbs, "frac": gbs / peak,
            "kernel": KERNEL_NAMES.get(info["kernel_last"], str(info["kernel_last"])),
            "note": f"config 4 at {B} of its 131072 rows (host generation of the full batch is ~20 GB)",
            "mapping": mapping}


def perop_baseline(w, host, dev, kern_ms, steps=10):
    """The paper's Sequential arm on this GPU (baselines/perop_torch.py): every
    graph node as its own eager PyTorch operation(s), intermediates in HBM;
    inputs resident, CUDA events around whole-graph evaluations."""
    import torch

    from baselines.perop_torch import PerOpGraph

    g = PerOpGraph(w.spec, dev)
    b = g.upload(host)
    for _ in range(2):
        g.run(b)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        g.run(b)
    e1.record()
    e1.synchronize()
    ms = e0.elapsed_time(e1) / steps
    del b
    torch.cuda.empty_cache()
    return {"ms_per_step": ms, "fused_speedup": ms / kern_ms,
            "note": "one eager PyTorch evaluation per graph node (TorchArrow-style), same batch, "
                    "outputs equal to the oracle (tests/test_perop_baseline.py)"}


def plan_point(dev, plan_id, B, steps=20):
    """Table 3 Plan 2 / Plan 3-shaped graph (synth.plan_graph, 384 / 1548 ops)
    at B rows: kernel time (AUTO kernel choice), HBM fraction of the launch."""
    import torch

    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth

    w = synth.plan_graph(plan_id, 0)
    plan = rap.Plan(w.spec, device=dev.index)
    sets = []
    for i in range(2):
        h = synth.make_batch(w, B, seed=800 + i)
        r = rap.DeviceBatch(h, dev)
        sets.append((h, r, rap.DeviceOutput(plan, B, r.sp_nnz, dev)))
    stream = torch.cuda.current_stream(dev)
    for i in range(4):
        plan.preprocess(sets[i % 2][1], sets[i % 2][2], stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for i in range(steps):
        plan.preprocess(sets[i % 2][1], sets[i % 2][2], stream)
    e1.record(stream)
    e1.synchronize()
    ms = e0.elapsed_time(e1) / steps
    last = sets[(steps - 1) % 2]
    n_vals = int(last[2].offsets[-1].item())
    alg = synth.algorithmic_bytes(w.spec, last[0], n_vals)
    peak, _ = measured_peaks()
    info = plan.info()
    d_out, f_out = synth.output_dims(w.spec)
    plan.close()
    del sets
    torch.cuda.empty_cache()
    gbs = alg / (ms / 1e3) / 1e9
    return {"workload": w.name, "graph_ops": len(w.spec["nodes"]), "dense_out_cols": d_out,
            "sparse_out_features": f_out, "batch": B, "kernel_ms": ms, "value": B / (ms / 1e3), "unit": UNIT,
            "alg_bytes_per_launch": int(alg), "achieved_gbs": gbs, "frac": gbs / peak,
            "kernel": KERNEL_NAMES.get(info["kernel_last"], str(info["kernel_last"]))}


def step_graphs(plan, sets, K, stream):
    """CUDA graphs of the timed steps: g_full = one rap_preprocess launch per
    rotating set (<= 8: the plan caches 8 batch shapes' partitions and an
    eviction would sync the stream inside the capture), replayed K // n times,
    and g_rem = the first K % n launches (None if 0)."""
    import torch

    sets = sets[:8]
    n = len(sets)
    s = torch.cuda.Stream(stream.device)
    s.wait_stream(stream)
    with torch.cuda.stream(s):
        for r, o in sets:
            plan.preprocess(r, o, stream=s)  # every batch shape's partition cached
    s.synchronize()
    g_full = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g_full, stream=s):
        for r, o in sets:
            plan.preprocess(r, o, stream=s)
    g_rem = None
    if K % n:
        g_rem = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g_rem, stream=s):
            for r, o in sets[: K % n]:
                plan.preprocess(r, o, stream=s)
    for _ in range(2):
        g_full.replay()
    torch.cuda.synchronize()
    return g_full, K // n, g_rem


def graph_replay(plan, sets, B, dev, steps, alg_bytes):
    """The same launches captured once in a CUDA graph (one rap_preprocess per
    rotating input/output set) and replayed: removes the per-call host cost
    (ctypes marshalling, C-ABI validation) that bounds small batches (C1).
    Same kernel, same inputs and outputs; reported beside the per-call line."""
    import torch

    # the plan caches 8 batch shapes' work partitions and evicting one syncs the
    # stream (illegal during capture), so the graph covers at most 8 sets
    sets = sets[:8]
    nsets = len(sets)
    s = torch.cuda.Stream(dev)
    with torch.cuda.stream(s):
        for r, o in sets:
            plan.preprocess(r, o, stream=s)  # warm-up: every batch shape's partition cached
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for r, o in sets:
            plan.preprocess(r, o, stream=s)
    reps = max(1, steps // nsets)
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record()
    for _ in range(reps):
        g.replay()
    t1.record()
    t1.synchronize()
    ms = t0.elapsed_time(t1) / (reps * nsets)
    o = sets[-1][1]
    assert int(o.offsets[0]) == 0 and bool((o.offsets[1:] >= o.offsets[:-1]).all())
    return {"ms_per_step": ms, "value": B / (ms / 1e3), "unit": UNIT, "launches": reps * nsets,
            "what": f"CUDA graph of {nsets} rap_preprocess launches (one per rotating set), replayed {reps}x",
            "l2_policy": f"rotate {nsets} sets, {nsets * alg_bytes / 2**20:.0f} MB"}


def fusion_ablation(w, sets, B, dev, stream, fused_ms, steps):
    """"RAP w/o fusion" analog (Fig 10 ablation): the same graph
    run as one launch per output feature (each its own single-output plan, the
    features executed back to back on one stream) instead of one horizontally fused
    launch.  Same kernel code and inputs; only the fusion differs.  Reported as
    context next to the paper's 1.15x (w/o fusion vs full RAP is not printed as a
    ratio there)."""
    import torch

    from paper_conf_asplos_wangwdz0d24_b200 import rap

    plans = []
    for o in w.spec["outputs"]:
        s = dict(w.spec)
        s["outputs"] = [o]
        p = rap.Plan(s, device=dev.index)
        p.set_kernel(rap.KERNEL_ROWS)  # one-output launches: the interpreted row-block kernel (no NVRTC per plan)
        plans.append(p)
    nsets = len(sets)
    outs = [[rap.DeviceOutput(p, B, r.sp_nnz, dev) for p in plans] for r, _ in sets]

    def one(i):
        r = sets[i % nsets][0]
        for p, o in zip(plans, outs[i % nsets]):
            p.preprocess(r, o, stream)

    for i in range(5):
        one(i)
    torch.cuda.synchronize()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record(stream)
    for i in range(steps):
        one(i)
    t1.record(stream)
    t1.synchronize()
    unfused_ms = t0.elapsed_time(t1) / steps
    for p in plans:
        p.close()
    del outs
    torch.cuda.empty_cache()
    return {"fused_ms": fused_ms, "unfused_ms": unfused_ms, "launches_unfused": len(plans),
            "fusion_speedup": unfused_ms / fused_ms, "steps": steps,
            "what": "one fused launch (the timed kernel) vs one launch per output feature (interpreted row-block "
                    "kernel, same inputs)"}


def run_sharded(args):
    """N > 1 (config 3): the C2 graph feature-sharded across the ranks with
    table-wise placement.  Global batch fixed -> strong scaling;
    value = global rows / max-over-ranks step time (residual exchange included)."""
    import torch
    import torch.distributed as tdist

    rank, world, local = dist_env()
    local = local % max(torch.cuda.device_count(), 1)  # gloo test runs: several ranks may share a GPU
    torch.cuda.set_device(local)
    if args.dist_backend == "nccl":
        tdist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        tdist.init_process_group("gloo")
    dev = torch.device("cuda", local)
    from paper_conf_asplos_wangwdz0d24_b200 import dist, rap, synth

    exchange = None if args.dist_backend == "nccl" else dist.gloo_exchange

    wname, B = WORKLOADS[args.workload]
    B = args.batch or B
    w = workload(args.workload)
    host = synth.make_batch(w, B, seed=1000)  # the global batch (each rank uploads its own part of it)
    sp_nnz = np.array([int(o[-1]) - int(o[0]) for o in host["sp_off"]], dtype=np.int64)
    comm = calibrate_comm(w.spec, host, B, dev, tdist)
    pl = dist.plan_placement(w.spec, B, sp_nnz, world, args.placement, args.imbalance_tol, device=local, comm=comm)
    sp = dist.ShardedPreprocessor(w.spec, pl, rank, world, B, sp_nnz, device=local, sm_budget=args.budget)
    cols = sp.sparse_columns()
    nsets = 1 if args.profile else 4
    sets = []
    for i in range(nsets):
        h = host if i == 0 else synth.make_batch(w, B, seed=1000 + 97 * i)
        r = rap.DeviceBatch(h, dev, sparse_cols=cols, dense_rows=(sp.row0, sp.dense_rows))
        sets.append((r, sp.new_output()))
    upload = sets[0][0].uploaded_bytes()
    stream = torch.cuda.current_stream(dev)
    for i in range(args.warmup):
        r, o = sets[i % nsets]
        sp.preprocess(r, o, stream, exchange=exchange)
    torch.cuda.synchronize()
    tdist.barrier()
    torch.cuda.synchronize()
    K = args.steps
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(local) if not args.profile else None
    with (sampler if sampler else _Null()):
        t0.record(stream)
        for i in range(K):
            r, o = sets[i % nsets]
            sp.preprocess(r, o, stream, exchange=exchange)
        t1.record(stream)
        t1.synchronize()
    torch.cuda.synchronize()
    tdist.barrier()
    total_ms = allreduce_max(t0.elapsed_time(t1), dev, tdist)
    # my share of the algorithmic bytes: owned tables over the full batch + my dense shard
    o = sets[(K - 1) % nsets][1]
    offs = o.offsets
    assert int(offs[0]) == 0 and bool((offs[1:] >= offs[:-1]).all())
    n_vals = int(offs[-1].item())
    d_out = sp.d_out
    my_bytes = (4 * sp.dense_rows * d_out + len(sp.features) * B * 20 + 8 * n_vals
                + (13 * 4.125 * sp.dense_rows if d_out else 0))
    bt = [allreduce_max(my_bytes, dev, tdist)]
    peak, peak_kind = measured_peaks()
    ms = total_ms / K
    achieved = float(bt[0]) / (ms / 1e3) / 1e9
    clocks = sampler.summary() if sampler else None
    c4 = None if (args.no_c4 or args.profile) else c4_sharded_point(args, rank, world, dev, tdist, exchange)
    if rank == 0:
        res = pl.residual
        line = {"metric": METRIC, "value": B / (ms / 1e3), "unit": UNIT, "n_gpus": world, "steps": K,
                "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": "int64+f32", "data": "synthetic",
                "config": {"workload": wname + "_sharded_c3", "batch": B, "parallelism": f"table-wise x{world}",
                           "placement": args.placement, "loads": [round(x) for x in pl.loads],
                           "residual": None if res is None else res.__dict__,
                           "comm_model": comm.__dict__,
                           "rank0_upload_bytes": upload, "rank0_sparse_columns": len(cols),
                           "l2_policy": f"rotate {nsets} input/output sets"},
                "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                             "frac": achieved / peak, "traffic": None, "peak_source": peak_kind,
                             "note": "busiest rank's algorithmic bytes / step time"},
                "cpu_baseline": None, "e2e": None, "clocks": clocks,
                "gpu_launches": K * (1 + (0 if res is None else 2)), "c4": c4}
        print(json.dumps(line), flush=True)
    sp.close()
    tdist.destroy_process_group()
    return 0


def allreduce_max(x: float, dev, tdist) -> float:
    """Max over ranks of a host scalar (a CUDA tensor over NCCL, a CPU one over gloo)."""
    import torch

    on_gpu = tdist.get_backend() == "nccl"
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev if on_gpu else "cpu")
    tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    return float(t[0])


def calibrate_comm(spec, host, B, dev, tdist):
    """rap_comm_model's time scale on this GPU: rank 0 times the full plan on
    the batch and divides by its predicted cost (broadcast, so every rank
    computes the same placement)."""
    import torch

    from paper_conf_asplos_wangwdz0d24_b200 import dist, rap

    t = torch.zeros(1, dtype=torch.float64, device=dev if tdist.get_backend() == "nccl" else "cpu")
    if tdist.get_rank() == 0:
        plan = rap.Plan(spec, device=dev.index)
        raw = rap.DeviceBatch(host, dev)
        out = rap.DeviceOutput(plan, B, raw.sp_nnz, dev)
        for _ in range(3):
            plan.preprocess(raw, out)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10):
            plan.preprocess(raw, out)
        e1.record()
        e1.synchronize()
        us = e0.elapsed_time(e1) / 10 * 1e3
        t[0] = us / max(float(sum(plan.output_costs(B, raw.sp_nnz))), 1e-9)
        plan.close()
        del raw, out
    tdist.broadcast(t, 0)
    return dist.CommModel(us_per_unit=float(t[0]))


def c4_sharded_point(args, rank, world, dev, tdist, exchange=None):
    """Config 4 table-wise over the ranks (512 tables, balanced, no residual):
    each rank uploads and preprocesses its own tables over the global batch;
    the step time is the max over ranks."""
    import torch

    from paper_conf_asplos_wangwdz0d24_b200 import dist, rap, synth

    w = synth.c4_multihot(0)
    B = args.c4_batch
    host = synth.make_batch(w, B, seed=700)
    sp_nnz = np.array([int(o[-1]) - int(o[0]) for o in host["sp_off"]], dtype=np.int64)
    pl = dist.plan_placement(w.spec, B, sp_nnz, world, "balanced", None, device=dev.index)
    sp = dist.ShardedPreprocessor(w.spec, pl, rank, world, B, sp_nnz, device=dev.index)
    raw = rap.DeviceBatch(host, dev, sparse_cols=sp.sparse_columns())
    out = sp.new_output()
    stream = torch.cuda.current_stream(dev)
    for _ in range(3):
        sp.preprocess(raw, out, stream, exchange=exchange)
    torch.cuda.synchronize()
    tdist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    steps = 10
    e0.record(stream)
    for _ in range(steps):
        sp.preprocess(raw, out, stream, exchange=exchange)
    e1.record(stream)
    e1.synchronize()
    ms = allreduce_max(e0.elapsed_time(e1) / steps, dev, tdist)
    sp.close()
    del raw, out
    torch.cuda.empty_cache()
    return {"workload": "multihot_c4_sharded", "batch": B, "tables_per_rank": len(sp.features),
            "ms_per_step": ms, "value": B / (ms / 1e3), "unit": UNIT, "scaling": "strong",
            "note": "table-wise over the ranks, global batch fixed; max over ranks"}


class _Null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    return run_rap(args)


if __name__ == "__main__":
    sys.exit(main())
