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

    def step(self):
        """Forward, backward, SGD (MLP weights and the gathered embedding rows)."""
        import torch

        x = self.dense
        for i, w in enumerate(self.bot):
            x = x @ w.t()
            x = torch.relu(x) if i < len(self.bot) - 1 else x
        embs = [t.index_select(0, i).to(torch.bfloat16).requires_grad_() for t, i in zip(self.tables, self.idx)]
        feats = torch.stack([x] + embs, dim=1)                        # [B, 27, dim]
        inter = torch.bmm(feats, feats.transpose(1, 2))[:, self.iu[0], self.iu[1]]
        z = torch.cat([x, inter], dim=1)
        for i, w in enumerate(self.top):
            z = z @ w.t()
            z = torch.relu(z) if i < len(self.top) - 1 else z
        loss = torch.nn.functional.binary_cross_entropy_with_logits(z.float(), self.label.float())
        params = self.bot + self.top
        grads = torch.autograd.grad(loss, params + embs)
        with torch.no_grad():
            for p, gr in zip(params, grads[: len(params)]):
                p.sub_(self.lr * gr)
            for t, i, gr in zip(self.tables, self.idx, grads[len(params):]):
                t.index_add_(0, i, gr.float(), alpha=-self.lr)
        return loss


def measure(plan, sets, train: DLRMStep, budgets, steps=20, warmup=5):
    """Per budget: training step alone vs co-run with one preprocessing launch
    per step (events on each stream), in ms, and the slowdown."""
    import torch

    hi = torch.cuda.Stream(priority=-1)  # training: highest priority
    lo = torch.cuda.Stream(priority=0)   # preprocessing: lowest
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731

    def run(k, with_prep, with_train=True):
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
    for b in budgets:
        plan.set_budget(b)
        run(warmup, True)
        _, prep_alone = run(steps, True, with_train=False)
        t, p = run(steps, True)
        res["per_budget"].append({"sm_budget": b, "train_step_corun_ms": t, "prep_corun_ms": p,
                                  "prep_alone_ms": prep_alone, "slowdown": t / alone - 1.0,
                                  "prep_hidden": p <= t})
    plan.set_budget(0)
    return res
