"""Co-run measurement (§3, §6.2).

A synthetic DLRM training step (the workload RAP shares the GPU with) runs on
a high-priority stream while the fused preprocessing of the NEXT batch runs
under an SM budget on a low-priority stream.  Reported: the training step
alone and co-run (CUDA events on the training stream), the preprocessing
latency co-run, and slowdown = T_corun / T_alone - 1.

The training step is plain PyTorch (cuBLAS GEMMs + embedding gather /
index_add_): it is the co-runner being protected, not part of the method.
Shape (DESIGN.md §3 A19): 26 tables x dim 128 fp32, the per-GPU share of
the Terabyte tables at 8 GPUs (sum 177.9M rows / 8), local batch 8192,
bottom MLP 13-512-256-128, dot interaction 27*26/2 + 128 = 479, top MLP
479-1024-1024-512-256-1, bf16 MLP, SGD.
"""
from __future__ import annotations

import numpy as np


class DLRMStep:
    def __init__(self, device, batch=8192, table_rows=None, dim=128, n_tables=26, seed=0, lr=0.01):
        import torch

        g = torch.Generator(device="cpu").manual_seed(seed)
        self.dev, self.B, self.dim, self.T, self.lr = device, batch, dim, n_tables, lr
        if table_rows is None:
            # per-GPU share of the Terabyte tables under table-wise sharding at 8 GPUs
            from . import synth

            M = synth.cardinalities(0, n_tables, synth.TB_TOTAL)
            table_rows = [max(int(m) // 8, 16) for m in M]
        self.rows = table_rows
        self.tables = [torch.empty(r, dim, device=device).uniform_(-0.01, 0.01) for r in table_rows]

        def lin(i, o):
            w = (torch.randn(o, i, generator=g) / np.sqrt(i)).to(device=device, dtype=torch.bfloat16)
            return w.requires_grad_()

        self.bot = [lin(13, 512), lin(512, 256), lin(256, dim)]
        n_int = (n_tables + 1) * n_tables // 2 + dim
        self.top = [lin(n_int, 1024), lin(1024, 1024), lin(1024, 512), lin(512, 256), lin(256, 1)]
        self.dense = torch.randn(batch, 13, generator=g).to(device=device, dtype=torch.bfloat16)
        self.idx = [torch.randint(0, r, (batch,), generator=g).to(device) for r in table_rows]
        self.label = torch.randint(0, 2, (batch, 1), generator=g).to(device=device, dtype=torch.bfloat16)
        iu = torch.triu_indices(n_tables + 1, n_tables + 1, 1)
        self.iu = (iu[0].to(device), iu[1].to(device))

    LAYERS = ("bottom_mlp", "embedding", "interaction", "top_mlp", "backward", "update")

    def step(self, hook=None):
        """Forward, backward, SGD (MLP weights and the gathered embedding rows).
        hook(layer) is called on the training stream as each layer begins
        (layer-aligned co-run scheduling, §7.1)."""
        import torch

        h = hook or (lambda name: None)
        h("bottom_mlp")
        x = self.dense
        for i, w in enumerate(self.bot):
            x = x @ w.t()
            x = torch.relu(x) if i < len(self.bot) - 1 else x
        h("embedding")
        embs = [t.index_select(0, i).to(torch.bfloat16).requires_grad_() for t, i in zip(self.tables, self.idx)]
        h("interaction")
        feats = torch.stack([x] + embs, dim=1)                        # [B, 27, dim]
        inter = torch.bmm(feats, feats.transpose(1, 2))[:, self.iu[0], self.iu[1]]
        z = torch.cat([x, inter], dim=1)
        h("top_mlp")
        for i, w in enumerate(self.top):
            z = z @ w.t()
            z = torch.relu(z) if i < len(self.top) - 1 else z
        loss = torch.nn.functional.binary_cross_entropy_with_logits(z.float(), self.label.float())
        h("backward")
        params = self.bot + self.top
        grads = torch.autograd.grad(loss, params + embs)
        h("update")
        with torch.no_grad():
            for p, gr in zip(params, grads[: len(params)]):
                p.sub_(self.lr * gr)
            for t, i, gr in zip(self.tables, self.idx, grads[len(params):]):
                t.index_add_(0, i, gr.float(), alpha=-self.lr)
        h(None)
        return loss

    def layer_times_us(self, steps=10):
        """Median duration of every layer of the step run alone (events on the
        stream): the windows the layer-aligned schedule fills."""
        import torch

        per = {n: [] for n in self.LAYERS}
        for _ in range(steps + 2):
            evs = []

            def hook(name):
                e = torch.cuda.Event(enable_timing=True)
                e.record()
                evs.append((name, e))

            torch.cuda.synchronize()
            self.step(hook)
            torch.cuda.synchronize()
            for (n, a), (_, b) in zip(evs, evs[1:]):
                per[n].append(a.elapsed_time(b) * 1e3)
        return {n: float(np.median(v[2:])) for n, v in per.items()}


def measure(plan, sets, train: DLRMStep, budgets, steps=20, warmup=5, choose=None, partitions=()):
    """Per budget: training step alone vs co-run with one preprocessing launch
    per step (events on each stream), in ms, and the slowdown.  choose =
    (n_rows, sp_nnz): also the budget rap_choose_budget picks for an overlap
    capacity OC = the measured training step (the preprocessing of the next
    batch hides under one step, T_delta = P - OC <= 0, L1138-1152)."""
    import torch

    hi = torch.cuda.Stream(priority=-1)  # training: highest priority
    lo = torch.cuda.Stream(priority=0)   # preprocessing: lowest
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731

    def run(k, with_prep, with_train=True, lo=lo):
        t_train, t_prep = [], []
        for i in range(k):
            r, o = sets[i % len(sets)]
            a0, a1, b0, b1 = ev(), ev(), ev(), ev()
            torch.cuda.synchronize()
            if with_train:
                with torch.cuda.stream(hi):
                    a0.record(hi)
                    train.step()
                    a1.record(hi)
            if with_prep:
                b0.record(lo)
                plan.preprocess(r, o, lo)
                b1.record(lo)
            torch.cuda.synchronize()
            if with_train:
                t_train.append(a0.elapsed_time(a1))
            if with_prep:
                t_prep.append(b0.elapsed_time(b1))
        return (float(np.median(t_train)) if t_train else None, float(np.median(t_prep)) if t_prep else None)

    run(warmup, True)
    alone, _ = run(steps, False)
    res = {"train_step_alone_ms": alone, "per_budget": []}
    budgets = list(budgets)
    chosen = None
    if choose is not None:
        n_rows, nnz = choose
        oc_us = alone * 1e3
        b, td = plan.choose_budget(n_rows, nnz, oc_us)
        chosen = {"sm_budget": b, "overlap_capacity_us": oc_us, "predicted_us": plan.predict_latency_us(n_rows, nnz, b),
                  "t_delta_us": td}
        res["chosen"] = chosen
        if b not in budgets:
            budgets.append(b)
    def paired(lo_stream=lo):
        """Training alone and co-run measured in alternating rounds (medians),
        so clock / thermal drift over the sweep cancels in the slowdown."""
        ta, tc, pc = [], [], []
        for _ in range(4):
            ta.append(run(max(steps // 4, 3), False)[0])
            t_, p_ = run(max(steps // 4, 3), True, lo=lo_stream)
            tc.append(t_)
            pc.append(p_)
        return float(np.median(ta)), float(np.median(tc)), float(np.median(pc))

    for b in budgets:
        plan.set_budget(b)
        run(warmup, True)
        _, prep_alone = run(steps, True, with_train=False)
        alone_b, t, p = paired()
        res["per_budget"].append({"sm_budget": b, "train_step_alone_ms": alone_b, "train_step_corun_ms": t,
                                  "prep_corun_ms": p, "prep_alone_ms": prep_alone, "slowdown": t / alone_b - 1.0,
                                  "prep_hidden": p <= t, "chosen": chosen is not None and b == chosen["sm_budget"]})
        if chosen is not None and b == chosen["sm_budget"]:
            chosen.update({"measured_prep_alone_us": prep_alone * 1e3, "slowdown": t / alone_b - 1.0})
    # the same launches on a green-context SM partition (rap_sm_partition_stream):
    # the budget enforced by the hardware, not by the grid size
    from . import rap

    res["partition"] = []
    for b in partitions:
        part = rap.SMPartitionStream(torch.cuda.current_device(), b, priority=0)
        plan.set_budget(part.sms)
        run(warmup, True, lo=part.stream)
        _, prep_alone = run(steps, True, with_train=False, lo=part.stream)
        alone_b, t, p = paired(part.stream)
        res["partition"].append({"requested_sms": b, "partition_sms": part.sms, "train_step_alone_ms": alone_b,
                                 "train_step_corun_ms": t, "prep_corun_ms": p, "prep_alone_ms": prep_alone,
                                 "slowdown": t / alone_b - 1.0,
                                 "prep_hidden": p <= t})
        part.close()
    plan.set_budget(0)
    return res


# ------------------------------------------------- layer-aligned scheduling
class LayerAlignedPrep:
    """Layer-aligned co-run scheduling (§5.1, §7.1
    Algorithm 1): the plan's sparse outputs are cut into chunks
    (graph pieces, consecutive in output order; the dense outputs ride with
    the first) and each chunk is launched as its own fused kernel when a
    chosen training layer begins, on a low-priority stream, under the SM
    budget rap_choose_budget gives it for that layer's window (its overlap
    capacity OC_l, the layer's duration alone).  `budget` sets the SM count
    the greedy packs for (0 = all SMs).  Assignment is Algorithm 1's
    greedy: walk the layers in step order, give the current layer outputs
    while their predicted latency fits its remaining capacity, and when an
    output group does not fit, shard it -- the part that fits stays, the rest
    starts the next layer.  Chunks chain into ONE output (RAP_OUT_CHAIN), so
    the result equals the single fused launch (tests/test_gpu_corun.py)."""

    def __init__(self, spec, n_rows, sp_nnz, layer_us, device=0, order=None, min_chunk=2, budget=0):
        from . import dist, rap, synth

        self.B = n_rows
        self.layers = list(order or DLRMStep.LAYERS)
        full = rap.Plan(spec, device=device)
        types = synth.output_types(spec)
        sp_outs = [o for o, t in zip(spec["outputs"], types) if t == "I"]
        dn_outs = [o for o, t in zip(spec["outputs"], types) if t != "I"]
        costs = full.output_costs(n_rows, sp_nnz)
        # the greedy packs by the latency at `budget` SMs (0 = all): a small
        # budget spreads the chunks over more layers, each on fewer SMs
        p_full = full.predict_latency_us(n_rows, sp_nnz, budget)
        d_out, f_out, _ = full.output_shape(n_rows, sp_nnz)
        full.close()
        total = float(sum(costs)) or 1.0
        # Algorithm 1 (greedy over layers, shard on overflow): predicted
        # latency of a group ~ its share of the full plan's at all SMs
        share = [p_full * c / total for c in costs]
        cap = [float(layer_us[n]) for n in self.layers]
        assign, li, cur, used = [], 0, [], 0.0
        for j in range(len(sp_outs)):
            if cur and used + share[j] > cap[li] and len(cur) >= min_chunk and li + 1 < len(self.layers):
                assign.append((self.layers[li], cur))
                li, cur, used = li + 1, [], 0.0
            cur.append(j)
            used += share[j]
        if cur:
            assign.append((self.layers[li], cur))
        self.chunks = []
        slot = 0
        for k, (layer, js) in enumerate(assign):
            sub = dict(spec)
            sub["outputs"] = (dn_outs if k == 0 else []) + [sp_outs[j] for j in js]
            plan = rap.Plan(sub, device=device)
            oc = float(layer_us[layer])
            b, td = plan.choose_budget(n_rows, sp_nnz, oc)
            if budget > 0:  # never below the budget the chunk was packed for
                b = max(b, budget)
                td = plan.predict_latency_us(n_rows, sp_nnz, b) - oc
            plan.set_budget(b)
            self.chunks.append({"layer": layer, "outputs": js, "plan": plan, "slot": slot, "budget": b,
                                "oc_us": oc, "t_delta_us": td,
                                "predicted_us": plan.predict_latency_us(n_rows, sp_nnz, b)})
            slot += len(js)
        self.d_out, self.f_out = d_out, f_out
        self.features = list(range(len(sp_outs)))
        self._dist = dist

    def output(self, sp_nnz, device):
        vb = sum(c["plan"].output_shape(self.B, sp_nnz)[2] for c in self.chunks)
        return self._dist.RankOutput(self.features, self.B, self.B, self.d_out, vb, device)

    def launch(self, raw, out, stream, layer=None):
        """Launch the chunks assigned to `layer` (None: every chunk) on stream."""
        for c in self.chunks:
            if layer is None or c["layer"] == layer:
                c["plan"].preprocess_struct(raw.struct, out.struct(c["slot"], 0, chain=c["slot"] > 0), stream)

    def describe(self):
        return [{k: v for k, v in c.items() if k != "plan"} for c in self.chunks]

    def close(self):
        for c in self.chunks:
            c["plan"].close()


def measure_layer_aligned(lap: LayerAlignedPrep, sets_raw, outs, train: DLRMStep, steps=20, warmup=5):
    """Training step co-run with the layer-aligned chunks: each chunk's launch
    on the low-priority stream waits for an event recorded when its layer
    begins on the training stream.  Returns (co-run step, preprocessing done,
    the step alone measured in alternating rounds), medians in ms."""
    import torch

    rounds = [(_measure_la(lap, sets_raw, outs, train, max(steps // 4, 3), warmup if r == 0 else 1, False),
               _measure_la(lap, sets_raw, outs, train, max(steps // 4, 3), 1, True)) for r in range(4)]
    alone = float(np.median([a[0] for a, _ in rounds]))
    t = float(np.median([c[0] for _, c in rounds]))
    p = float(np.median([c[1] for _, c in rounds]))
    return t, p, alone


def _measure_la(lap, sets_raw, outs, train, steps, warmup, with_prep):
    import torch

    hi = torch.cuda.Stream(priority=-1)
    lo = torch.cuda.Stream(priority=0)
    t_train, t_prep = [], []
    assert len(sets_raw) == len(outs)  # output i sized for batch i
    for i in range(warmup + steps):
        raw, out = sets_raw[i % len(sets_raw)], outs[i % len(outs)]
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()

        def hook(name):
            if not with_prep or name is None or not any(c["layer"] == name for c in lap.chunks):
                return
            e = torch.cuda.Event()
            e.record(hi)
            lo.wait_event(e)
            lap.launch(raw, out, lo, name)

        with torch.cuda.stream(hi):
            a0.record(hi)
            p0.record(hi)
            train.step(hook)
            a1.record(hi)
        p1.record(lo)
        torch.cuda.synchronize()
        if i >= warmup:
            t_train.append(a0.elapsed_time(a1))
            t_prep.append(p0.elapsed_time(p1))
    return float(np.median(t_train)), float(np.median(t_prep))
