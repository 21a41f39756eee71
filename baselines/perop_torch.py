"""Sequential per-op baseline on the GPU (the paper's
"Sequential" arm, Fig 10, and the unfused framing of L2238-2240):
every graph node is evaluated as its own eager PyTorch operation(s) over the
whole batch, each intermediate materialised in HBM, in topological order --
the way a per-op preprocessing library (TorchArrow-style) runs the same graph
on the same B200.  It is a measured comparison arm for bench.py, not part of
the product path (it never calls librap) and not a reference for parity: its
own test (tests/test_gpu_perop_baseline.py) checks it against the oracle.

Semantics are the DESIGN.md readings: R1-R3 SplitMix64 / multiply-high /
SigridHash (M < 2^32 here), R4 Bucketize (right side), R5 FirstX, R6 Clamp,
R7 NGram over the row-wise concatenation, R8 MapId, R9 OneHot, R10 FillNull,
R11 Logit, R12 BoxCox, R14 nulls, R17 output layout.

A list value is (lengths int64[B], offsets int64[B+1] from 0, values
int64[total], null bool[B]); a dense value is f32[B] (NaN = null, R14).
"""
from __future__ import annotations

import numpy as np
import torch

M64 = (1 << 64) - 1


def _i64(x: int) -> int:
    """Two's-complement int64 view of an unsigned 64-bit constant."""
    x &= M64
    return x - (1 << 64) if x >= 1 << 63 else x


def _srl(z: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (z >> s) & ((1 << (64 - s)) - 1)


_G, _C1, _C2 = _i64(0x9E3779B97F4A7C15), _i64(0xBF58476D1CE4E5B9), _i64(0x94D049BB133111EB)


def H(x: torch.Tensor) -> torch.Tensor:
    """R1 SplitMix64 on int64 bit patterns (wrapping multiply)."""
    z = x + _G
    z = (z ^ _srl(z, 30)) * _C1
    z = (z ^ _srl(z, 27)) * _C2
    return z ^ _srl(z, 31)


def H_scalar(x: int) -> int:
    z = (x + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def reduce_M(h: torch.Tensor, M: int) -> torch.Tensor:
    """R2 floor(h * M / 2^64) for M < 2^32 in 64-bit wrapping arithmetic:
    (hi * M + (lo * M >> 32)) >> 32, every product < 2^64 unsigned."""
    assert 0 < M < (1 << 32), "the baseline covers table sizes < 2^32"
    hi, lo = _srl(h, 32), h & 0xFFFFFFFF
    return _srl(hi * M + _srl(lo * M, 32), 32)


class Lst:
    __slots__ = ("L", "O", "V", "null")

    def __init__(self, L, V, null):
        self.L, self.V, self.null = L, V, null
        self.O = torch.zeros(L.numel() + 1, dtype=torch.int64, device=L.device)
        torch.cumsum(L, 0, out=self.O[1:])


def _rows_pos(L: torch.Tensor, O: torch.Tensor):
    """Row id and in-row position of every element of a list of lengths L."""
    B = L.numel()
    row = torch.repeat_interleave(torch.arange(B, device=L.device), L)
    pos = torch.arange(row.numel(), device=L.device) - O[:-1][row]
    return row, pos


def _sparse_input(off, val, valid, B):
    """Raw Arrow column -> list (null rows empty, R14)."""
    off = off.to(torch.int64)
    L = off[1:] - off[:-1]
    null = ~valid if valid is not None else torch.zeros(B, dtype=torch.bool, device=off.device)
    L = torch.where(null, torch.zeros_like(L), L)
    out = Lst(L, None, null)
    row, pos = _rows_pos(L, out.O)
    out.V = val[off[:-1][row] + pos]
    return out


def _bits_to_bool(words, B):
    w = words.to(torch.int64) & 0xFFFFFFFF
    b = (w.unsqueeze(1) >> torch.arange(32, device=w.device)) & 1
    return b.reshape(-1)[:B].bool()


class PerOpGraph:
    """One eager PyTorch evaluation per node (bench.py's per-op arm)."""

    def __init__(self, spec, device):
        self.spec, self.dev = spec, torch.device(device)
        self.types = {}
        self.tabs = {}
        for i, nd in enumerate(spec["nodes"]):
            if nd["op"] == "mapid":
                k = np.asarray(nd["keys"], dtype=np.int64)
                v = np.asarray(nd["vals"], dtype=np.int64)
                o = np.argsort(k, kind="stable")
                self.tabs[i] = (torch.from_numpy(k[o]).to(self.dev), torch.from_numpy(v[o]).to(self.dev))
            elif nd["op"] == "bucketize":
                b = np.asarray(nd["borders"])
                self.tabs[i] = torch.from_numpy(b.astype(np.float32 if b.dtype.kind == "f" else np.int64)).to(self.dev)
        self.hsalt = {i: _i64(H_scalar(int(nd["salt"]) & M64)) for i, nd in enumerate(spec["nodes"])
                      if nd["op"] in ("sigridhash", "ngram")}

    def upload(self, batch):
        """Host batch -> device tensors (the baseline's inputs, resident in HBM)."""
        d = self.dev
        t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a, dtype=dt)).to(d)  # noqa: E731
        return {"n_rows": int(batch["n_rows"]),
                "dense": [t(x, np.float32) for x in batch["dense"]],
                "dense_valid": [None if v is None else t(v, np.uint32).view(torch.int32) for v in batch["dense_valid"]],
                "sp_off": [t(o, np.int32) for o in batch["sp_off"]],
                "sp_val": [t(v, np.int64) if len(v) else torch.zeros(1, dtype=torch.int64, device=d)
                           for v in batch["sp_val"]],
                "sp_valid": [None if v is None else t(v, np.uint32).view(torch.int32) for v in batch["sp_valid"]]}

    def run(self, b):
        B = b["n_rows"]
        vals = {}

        def get(kind, idx):
            key = (kind, idx)
            if key in vals:
                return vals[key]
            if kind == "d":
                x = b["dense"][idx]
                v = b["dense_valid"][idx]
                if v is not None:
                    x = torch.where(_bits_to_bool(v, B), x, torch.full_like(x, float("nan")))
                vals[key] = x
            else:
                v = b["sp_valid"][idx]
                vals[key] = _sparse_input(b["sp_off"][idx], b["sp_val"][idx],
                                          None if v is None else _bits_to_bool(v, B), B)
            return vals[key]

        for i, nd in enumerate(self.spec["nodes"]):
            ins = [get(k, x) if k != "n" else vals[("n", x)] for k, x in nd["inputs"]]
            vals[("n", i)] = self._op(i, nd, ins, B)
        return self._assemble(vals, B)

    def _op(self, i, nd, ins, B):
        op, a = nd["op"], ins[0]
        if op == "fillnull":
            if isinstance(a, torch.Tensor):  # R10 dense
                return torch.where(torch.isnan(a), torch.full_like(a, float(nd["f_fill"])), a)
            L = torch.where(a.null, torch.ones_like(a.L), a.L)  # R10 sparse: null -> [fill]
            out = Lst(L, None, torch.zeros_like(a.null))
            row, pos = _rows_pos(L, out.O)
            src = a.V[(a.O[:-1][row] + pos).clamp(max=max(a.V.numel() - 1, 0))] if a.V.numel() else \
                torch.zeros_like(row)
            out.V = torch.where(a.null[row], torch.full_like(src, int(nd["i_fill"])), src)
            return out
        if op == "logit":  # R11 torch.logit
            return torch.logit(a, eps=float(nd["eps"]))
        if op == "boxcox":  # R12
            lam = float(nd["lambda"])
            return torch.log(a) if lam == 0.0 else torch.expm1(lam * torch.log(a)) / np.float32(lam)
        if op == "bucketize":  # R4
            bt = self.tabs[i]
            if isinstance(a, torch.Tensor):
                ids = torch.searchsorted(bt, torch.nan_to_num(a, nan=-float("inf")).contiguous(), right=True)
                ids = torch.where(torch.isnan(a), torch.zeros_like(ids), ids)
                return Lst(torch.ones(B, dtype=torch.int64, device=a.device), ids.to(torch.int64),
                           torch.zeros(B, dtype=torch.bool, device=a.device))
            out = Lst(a.L, torch.searchsorted(bt, a.V, right=True), a.null)
            return out
        if op == "onehot":  # R9
            K = int(nd["k"])
            row, _ = _rows_pos(a.L, a.O)
            m = (a.V >= 0) & (a.V < K)
            vec = torch.zeros(B, K, dtype=torch.float32, device=a.L.device)
            vec[row[m], a.V[m]] = 1.0
            return vec
        if op == "clamp":  # R6
            return Lst(a.L, a.V.clamp(int(nd["lo"]), int(nd["hi"])), a.null)
        if op == "sigridhash":  # R3
            return Lst(a.L, reduce_M(H(self.hsalt[i] ^ a.V), int(nd["max_value"])), a.null)
        if op == "mapid":  # R8
            k, v = self.tabs[i]
            j = torch.searchsorted(k, a.V).clamp(max=k.numel() - 1)
            hit = k[j] == a.V
            return Lst(a.L, torch.where(hit, v[j], torch.full_like(a.V, int(nd["map_default"]))), a.null)
        if op == "firstx":  # R5
            L = a.L.clamp(max=int(nd["x"]))
            out = Lst(L, None, a.null)
            row, pos = _rows_pos(L, out.O)
            out.V = a.V[a.O[:-1][row] + pos]
            return out
        if op == "ngram":  # R7: windows over the row-wise concatenation
            n = int(nd["n"])
            Ls = [torch.where(s.null, torch.zeros_like(s.L), s.L) for s in ins]
            C = torch.stack(Ls).sum(0)
            cat = Lst(C, None, torch.zeros(B, dtype=torch.bool, device=C.device))
            cat.V = torch.empty(int(cat.O[-1]), dtype=torch.int64, device=C.device)
            before = torch.zeros_like(C)
            for s, Ls_ in zip(ins, Ls):
                row, pos = _rows_pos(Ls_, s.O if s.V.numel() else s.O)
                cat.V[cat.O[:-1][row] + before[row] + pos] = s.V[s.O[:-1][row] + pos]
                before = before + Ls_
            W = (C - n + 1).clamp(min=0)
            out = Lst(W, None, torch.zeros(B, dtype=torch.bool, device=C.device))
            row, pos = _rows_pos(W, out.O)
            base = cat.O[:-1][row] + pos
            h = torch.full_like(base, self.hsalt[i])
            for t in range(n):
                h = H(h ^ cat.V[base + t])
            out.V = reduce_M(h, int(nd["max_value"]))
            return out
        raise ValueError(op)

    def _assemble(self, vals, B):
        """R17 layout: dense [B x D] in output order, KJT of the id lists."""
        dense, lists = [], []
        for o in self.spec["outputs"]:
            v = vals[("n", o)]
            if isinstance(v, Lst):
                lists.append(v)
            else:
                dense.append(v.reshape(B, -1))
        D = torch.cat(dense, 1) if dense else torch.zeros(B, 0, device=self.dev)
        if lists:
            lengths = torch.cat([torch.where(x.null, torch.zeros_like(x.L), x.L) for x in lists]).to(torch.int32)
            offsets = torch.zeros(lengths.numel() + 1, dtype=torch.int64, device=self.dev)
            torch.cumsum(lengths.to(torch.int64), 0, out=offsets[1:])
            values = torch.cat([x.V for x in lists])
        else:
            lengths = torch.zeros(0, dtype=torch.int32, device=self.dev)
            offsets = torch.zeros(1, dtype=torch.int64, device=self.dev)
            values = torch.zeros(0, dtype=torch.int64, device=self.dev)
        return {"dense": D, "lengths": lengths, "offsets": offsets, "values": values}
