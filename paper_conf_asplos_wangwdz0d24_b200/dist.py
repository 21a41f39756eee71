"""Multi-GPU RAP preprocessing (§7.2; hybrid parallelism
L488-499).

Table-wise, locality-aware: every sparse output (an embedding table) is
preprocessed over the FULL global batch on the rank that owns its table
(L1526-1534), so its KJT is already where the embedding lookup runs; dense
outputs are batch-sharded (each rank produces its own MLP mini-batch rows).
In the balanced case nothing moves.  When the placement leaves one rank above
the mean by more than a tolerance, a row range [split, B) of its costliest
output is preprocessed on the least loaded rank and shipped back (the paper's
residual redistribution, L1594-1600): the owner chains its own rows [0, split)
after its main launch (RAP_OUT_CHAIN) and appends the received piece with
rap_jagged_append, so its KJT is bit-identical to a single-GPU run.

This module is host orchestration.  Placement (rap_place), shard rows
(rap_shard_rows), the sharded plans, the fused kernel and the stitching all
run in librap; the piece transfer is NCCL point-to-point through
torch.distributed (plumbing), or an injected `exchange` callable.
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass

import numpy as np

from . import rap, synth


def sparse_output_nodes(spec) -> list:
    """Node index of every sparse output, in output order."""
    return [o for o, t in zip(spec["outputs"], synth.output_types(spec)) if t == "I"]


def _raw_sparse_source(spec, node):
    """Raw sparse column at the root of a node's first-input chain (None if dense)."""
    while True:
        kind, idx = spec["nodes"][node]["inputs"][0]
        if kind == "s":
            return idx
        if kind == "d":
            return None
        node = idx


def sparse_sources(spec, node) -> list:
    """Raw sparse columns a node reads (through every input, sorted)."""
    seen, out, stack = set(), set(), [node]
    while stack:
        n = stack.pop()
        if n in seen:
            continue
        seen.add(n)
        for kind, idx in spec["nodes"][n]["inputs"]:
            if kind == "s":
                out.add(idx)
            elif kind == "n":
                stack.append(idx)
    return sorted(out)


def row_bytes(spec, sp_nnz, n_rows: int) -> list:
    """Bytes one row of each sparse output moves in a residual exchange: its
    raw input row (offset, validity bit, ids of every source) to the helper and
    its output row (length, offset, ids -- bounded by the sources' ids) back."""
    B = max(int(n_rows), 1)
    out = []
    for n in sparse_output_nodes(spec):
        ids = sum(float(sp_nnz[c]) / B for c in sparse_sources(spec, n))
        srcs = len(sparse_sources(spec, n))
        out.append(srcs * (4 + 1 / 8) + 8 * ids + 12 + 8 * ids)
    return out


@dataclass
class CommModel:
    """rap_comm_model: cost-unit time scale and the owner <-> helper link."""
    us_per_unit: float
    link_gbs: float = 700.0        # NVLink 5 / NVSwitch point-to-point, effective
    link_latency_us: float = 20.0  # one NCCL send/recv pair: launch + synchronisation


def colocation(spec) -> list:
    """colocate[j] for the sparse outputs: an NGram table goes with the table
    of its first source column, -1 otherwise."""
    nodes = sparse_output_nodes(spec)
    first = {}
    col = []
    for j, n in enumerate(nodes):
        src = _raw_sparse_source(spec, n)
        if spec["nodes"][n]["op"] == "ngram":
            col.append(first.get(src, -1))
        else:
            col.append(-1)
            if src is not None and src not in first:
                first[src] = j
    return col


def shard_rows(n_rows: int, rank: int, world: int) -> tuple:
    r0, n = C.c_int64(), C.c_int64()
    rap._check(rap.load().rap_shard_rows(n_rows, rank, world, C.byref(r0), C.byref(n)))
    return r0.value, n.value


@dataclass
class Residual:
    output: int     # sparse output index
    owner: int
    helper: int
    split_row: int  # helper preprocesses rows [split_row, n_rows)


@dataclass
class Placement:
    owner: list
    loads: list
    residual: Residual | None
    mode: str


def place(costs, colocate, world: int, mode: str = "balanced", n_rows: int = 0, imbalance_tol: float | None = 0.1,
          comm: CommModel | None = None, row_bytes_=None):
    """rap_place (host only): table-wise owner of every sparse output, the
    predicted load per rank and the residual move (imbalance_tol None = never
    rebalance).  With a comm model (rap_place_comm) the move is made only when
    it shortens the owner's finish time after the exchange (L1594-1600)."""
    n = len(costs)
    c = np.ascontiguousarray(costs, dtype=np.float64)
    col = np.ascontiguousarray(colocate if colocate is not None else [-1] * n, dtype=np.int32)
    own = np.zeros(max(n, 1), dtype=np.int32)
    loads = np.zeros(world, dtype=np.float64)
    res = rap.RapResidual()
    L = rap.load()
    if comm is not None and imbalance_tol is not None:
        rb = np.ascontiguousarray(row_bytes_ if row_bytes_ is not None else [0.0] * n, dtype=np.float64)
        cm = rap.RapCommModel(comm.us_per_unit, comm.link_gbs, comm.link_latency_us, rb.ctypes.data if n else None)
        rap._check(L.rap_place_comm(c.ctypes.data if n else None, col.ctypes.data if n else None, n, world,
                                    rap.PLACE_MODES[mode], n_rows, C.byref(cm), own.ctypes.data, loads.ctypes.data,
                                    C.byref(res)))
    else:
        rap._check(L.rap_place(c.ctypes.data if n else None, col.ctypes.data if n else None, n, world,
                               rap.PLACE_MODES[mode], n_rows, 0.0 if imbalance_tol is None else imbalance_tol,
                               own.ctypes.data, loads.ctypes.data,
                               None if imbalance_tol is None else C.byref(res)))
    r = None
    if imbalance_tol is not None and res.output >= 0:
        r = Residual(res.output, res.owner, res.helper, res.split_row)
    return Placement([int(x) for x in own[:n]], [float(x) for x in loads], r, mode)


@dataclass
class JointMapping:
    owner: list    # rank evaluating each sparse output (-1: every rank, a duplicated graph)
    times: list    # per-rank time of the mapping (us): compute plus its exchanges
    moves: int     # substitutions made from the data-locality start


def place_joint(costs, colocate, home, world: int, n_rows: int, comm: CommModel, row_bytes_, oc_us: float = 0.0):
    """rap_place_joint (host only; §7.2): data-locality
    mapping (home[j]: the consumer rank of output j, -1 = duplicated on every
    rank), then substitutions of whole preprocessing graphs from the costliest
    to the cheapest rank while the co-running cost (largest exposed time over
    the overlap capacity oc_us, then the makespan) falls after charging the
    moved graph's input communication."""
    n = len(costs)
    c = np.ascontiguousarray(costs, dtype=np.float64)
    col = np.ascontiguousarray(colocate if colocate is not None else [-1] * n, dtype=np.int32)
    hm = np.ascontiguousarray(home, dtype=np.int32)
    rb = np.ascontiguousarray(row_bytes_ if row_bytes_ is not None else [0.0] * n, dtype=np.float64)
    cm = rap.RapCommModel(comm.us_per_unit, comm.link_gbs, comm.link_latency_us, rb.ctypes.data if n else None)
    own = np.zeros(max(n, 1), dtype=np.int32)
    times = np.zeros(world, dtype=np.float64)
    mv = C.c_int32()
    rap._check(rap.load().rap_place_joint(c.ctypes.data if n else None, col.ctypes.data if n else None,
                                          hm.ctypes.data if n else None, n, world, n_rows, C.byref(cm), float(oc_us),
                                          own.ctypes.data, times.ctypes.data, C.byref(mv)))
    return JointMapping([int(x) for x in own[:n]], [float(x) for x in times], int(mv.value))


def plan_placement(spec, n_rows: int, sp_nnz, world: int, mode: str = "balanced", imbalance_tol=0.1,
                   device: int = 0, comm: CommModel | None = None) -> Placement:
    """Placement from the plan's own cost model (rap_plan_output_costs);
    comm: cost the residual move's exchange (rap_place_comm)."""
    full = rap.Plan(spec, device=device)
    try:
        costs = full.output_costs(n_rows, sp_nnz)
    finally:
        full.close()
    return place(costs, colocation(spec), world, mode, n_rows, imbalance_tol, comm,
                 row_bytes(spec, sp_nnz, n_rows) if comm is not None else None)


class RankOutput:
    """One rank's outputs: dense rows of its batch shard, and a KJT of its
    features (`features`: sparse output indices in KJT order)."""

    def __init__(self, features, n_rows, dense_rows, d_out, values_cap, device):
        import torch

        F = len(features)
        self.features, self.n_rows, self.dense_rows, self.d_out = features, n_rows, dense_rows, d_out
        self.dense = torch.empty(max(dense_rows * d_out, 1), dtype=torch.float32, device=device)
        self.lengths = torch.empty(max(F * n_rows, 1), dtype=torch.int32, device=device)
        self.offsets = torch.empty(F * n_rows + 1, dtype=torch.int64, device=device)
        self.values = torch.empty(max(values_cap, 1), dtype=torch.int64, device=device)
        self.values_cap = values_cap

    def struct(self, feature_slot=0, row=0, chain=False):
        """RapOutput whose lengths/offsets start at (feature_slot, row)."""
        k = feature_slot * self.n_rows + row
        return rap.RapOutput(self.dense.data_ptr(), self.d_out, self.lengths.data_ptr() + 4 * k,
                             self.offsets.data_ptr() + 8 * k, self.values.data_ptr(), self.values_cap,
                             rap.RAP_OUT_CHAIN if chain else 0, 0)

    def to_numpy(self):
        F, B = len(self.features), self.n_rows
        off = self.offsets.cpu().numpy()
        return {"dense": self.dense.cpu().numpy()[: self.dense_rows * self.d_out].reshape(self.dense_rows, self.d_out),
                "lengths": self.lengths.cpu().numpy()[: F * B], "offsets": off,
                "values": self.values.cpu().numpy()[: int(off[-1])], "features": list(self.features)}


def nccl_exchange(rank: int, res: Residual, piece, recv_bufs, group=None):
    """Ship the residual piece helper -> owner with NCCL send/recv (the only
    data-path collective, L1594-1600).  piece / recv_bufs: [lengths, offsets,
    values] tensors of identical shapes on both sides."""
    import torch.distributed as dist

    ops = []
    if rank == res.helper:
        ops = [dist.P2POp(dist.isend, t, res.owner, group) for t in piece]
    elif rank == res.owner:
        ops = [dist.P2POp(dist.irecv, t, res.helper, group) for t in recv_bufs]
    if ops:
        for w in dist.batch_isend_irecv(ops):
            w.wait()


def gloo_exchange(rank: int, res: Residual, piece, recv_bufs, group=None):
    """The residual exchange staged through host memory over a CPU (gloo)
    group: ranks sharing one GPU (tests), where NCCL cannot run two ranks on
    one device.  Same protocol and buffers as nccl_exchange."""
    import torch
    import torch.distributed as dist

    if rank == res.helper:
        torch.cuda.synchronize()
        for t in piece:
            dist.send(t.cpu(), res.owner, group=group)
    elif rank == res.owner:
        for t in recv_bufs:
            h = torch.empty(t.shape, dtype=t.dtype)
            dist.recv(h, res.helper, group=group)
            t.copy_(h)


class ShardedPreprocessor:
    """One rank of the multi-GPU preprocessing."""

    def __init__(self, spec, placement: Placement, rank: int, world: int, n_rows: int, sp_nnz, device: int = 0,
                 sm_budget: int = 0):
        import torch

        self.spec, self.pl, self.rank, self.world, self.B = spec, placement, rank, world, n_rows
        self.dev = torch.device("cuda", device)
        sp_nodes = sparse_output_nodes(spec)
        res = placement.residual
        owner_main = list(placement.owner)
        if res is not None:
            owner_main[res.output] = -1
        self.main = rap.Plan.sharded(spec, owner_main, rank, world, device, sm_budget)
        self.main_features = [j for j, r in enumerate(owner_main) if r == rank]
        self.features = list(self.main_features)
        d_out, f_main, vb_main = self.main.output_shape(n_rows, sp_nnz)
        self.d_out = d_out
        self.row0, self.dense_rows = shard_rows(n_rows, rank, world)
        self.part = None
        cap = vb_main
        if res is not None and rank in (res.owner, res.helper):
            sub = dict(spec)
            sub["outputs"] = [sp_nodes[res.output]]
            self.part = rap.Plan(sub, device=device, sm_budget=sm_budget)
            n_hi = n_rows - res.split_row
            self.piece_bound = self.part.output_shape(n_hi, sp_nnz)[2]
            if rank == res.owner:
                self.features.append(res.output)
                cap += self.part.output_shape(res.split_row, sp_nnz)[2] + self.piece_bound
            else:
                self.piece = [torch.empty(max(n_hi, 1), dtype=torch.int32, device=self.dev),
                              torch.empty(n_hi + 1, dtype=torch.int64, device=self.dev),
                              torch.empty(max(self.piece_bound, 1), dtype=torch.int64, device=self.dev)]
            if rank == res.owner:
                self.recv = [torch.empty(max(n_hi, 1), dtype=torch.int32, device=self.dev),
                             torch.empty(n_hi + 1, dtype=torch.int64, device=self.dev),
                             torch.empty(max(self.piece_bound, 1), dtype=torch.int64, device=self.dev)]
        self.values_cap = cap

    def sparse_columns(self) -> list:
        """Raw sparse columns this rank reads: its own tables' (and the
        residual output's, on its owner and helper) -- what it uploads."""
        sp_nodes = sparse_output_nodes(self.spec)
        outs = list(self.main_features)
        res = self.pl.residual
        if res is not None and self.rank in (res.owner, res.helper):
            outs.append(res.output)
        cols = set()
        for j in outs:
            cols.update(sparse_sources(self.spec, sp_nodes[j]))
        return sorted(cols)

    def new_output(self) -> RankOutput:
        return RankOutput(self.features, self.B, self.dense_rows, self.d_out, self.values_cap, self.dev)

    def preprocess(self, raw: rap.DeviceBatch, out: RankOutput, stream=None, exchange=None):
        """Main launch (+ residual piece on the owner / helper, exchange, append)."""
        self.main.preprocess_struct(raw.struct, out.struct(0, 0), stream)
        res = self.pl.residual
        if self.part is None:
            return out
        n_hi = self.B - res.split_row
        if self.rank == res.helper:
            pv = rap.RapOutput(None, 0, self.piece[0].data_ptr(), self.piece[1].data_ptr(), self.piece[2].data_ptr(),
                               max(self.piece_bound, 0), 0, 0)
            self.part.preprocess_struct(rap.row_view(raw, res.split_row, n_hi), pv, stream)
        else:
            slot = len(self.main_features)  # slot 0: nothing precedes, the piece starts at 0
            self.part.preprocess_struct(rap.row_view(raw, 0, res.split_row),
                                        out.struct(slot, 0, chain=slot > 0), stream)
        ex = exchange or (lambda r, rs, piece, bufs: nccl_exchange(r, rs, piece, bufs))
        ex(self.rank, res, getattr(self, "piece", None), getattr(self, "recv", None))
        if self.rank == res.owner:
            k = len(self.main_features) * self.B + res.split_row
            rap._check(rap.load().rap_jagged_append(
                self.recv[0].data_ptr(), self.recv[1].data_ptr(), self.recv[2].data_ptr(), n_hi, self.piece_bound,
                out.lengths.data_ptr() + 4 * k, out.offsets.data_ptr() + 8 * k, out.values.data_ptr(),
                out.values_cap, rap._stream_handle(stream)))
        return out

    def close(self):
        self.main.close()
        if self.part is not None:
            self.part.close()
