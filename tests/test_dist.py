"""Multi-GPU path (§7.2).

CPU (`not gpu`): the host logic in librap (rap_place, rap_shard_rows) and the
residual protocol over a world_size-2 gloo group, where each rank's pieces
come from the oracle and the stitch is checked against the oracle's
single-process result.  GPU: every rank of a world W simulated on one B200
(sharded plans, chained launch, rap_jagged_append) must reproduce the
oracle's single-process result (ids bit-exact, dense within R16) and the
single-plan CUDA output bit for bit.
"""
import os
import socket

import numpy as np
import pytest

from paper_conf_asplos_wangwdz0d24_b200 import dist, rap, synth


# ----------------------------------------------------------------- host logic
def test_colocation_c2():
    w = synth.c2_terabyte(0)
    col = dist.colocation(w.spec)
    assert len(col) == 34 and col[:26] == [-1] * 26
    # trigram g reads sources 3g, 3g+1, 3g+2 (mod 26): it goes with table 3g
    assert col[26:] == [(3 * g) % 26 for g in range(8)]


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_shard_rows_partition(world):
    for B in (0, 1, 127, 128, 1000, 65536, 65537):
        spans = [dist.shard_rows(B, r, world) for r in range(world)]
        assert spans[0][0] == 0 and sum(n for _, n in spans) == B
        for (r0, n), (r1, _) in zip(spans, spans[1:]):
            assert r0 + n == r1 and r1 % 128 == 0 and n >= 0


def _costs(n, seed):
    rng = np.random.default_rng(seed)
    return rng.lognormal(0.0, 1.0, n) * 1000.0


@pytest.mark.parametrize("world", [2, 4, 8])
def test_place_balanced_lpt_bound(world):
    c = _costs(34, world)
    pl = dist.place(c, None, world, "balanced", 65536, None)
    loads = np.zeros(world)
    for j, r in enumerate(pl.owner):
        loads[r] += c[j]
    assert np.allclose(loads, pl.loads)
    # LPT: max load <= mean + largest item (Graham's bound)
    assert loads.max() <= c.sum() / world + c.max() + 1e-6


def test_place_round_robin_and_colocate():
    c = np.ones(10)
    col = [-1] * 8 + [0, 3]
    pl = dist.place(c, col, 4, "round_robin", 4096, None)
    groups = [j for j in range(10) if col[j] < 0]
    for i, j in enumerate(groups):
        assert pl.owner[j] == i % 4
    assert pl.owner[8] == pl.owner[0] and pl.owner[9] == pl.owner[3]


def test_place_skewed_and_residual():
    c = np.full(32, 100.0)
    pl = dist.place(c, None, 4, "skewed", 65536, None)
    loads = np.array(pl.loads)
    assert loads[0] == pytest.approx(2 * c.sum() / 4)  # rank 0 holds 2x the mean
    pr = dist.place(c, None, 4, "skewed", 65536, 0.1)
    r = pr.residual
    assert r is not None and r.owner == 0 and pr.owner[r.output] == 0
    assert r.helper != 0 and r.split_row % 128 == 0 and 128 <= r.split_row < 65536
    moved = (65536 - r.split_row) / 65536 * c[r.output]
    assert pr.loads[0] == pytest.approx(loads[0] - moved)
    assert max(pr.loads) < loads.max()
    # balanced placement of equal costs needs no residual
    assert dist.place(c, None, 4, "balanced", 65536, 0.1).residual is None


# ------------------------------------------------------- gloo residual protocol
def test_place_comm_moves_only_when_the_exchange_pays():
    """rap_place_comm (L1594-1600): a skewed placement moves rows only when the
    owner's finish time after the exchange beats keeping them; the chosen
    split balances compute against compute + transfer."""
    c = np.full(32, 100.0)
    B = 65536
    base = dist.place(c, None, 4, "skewed", B, None)
    L = np.array(base.loads)
    rb = [64.0] * 32
    # a fast link with little latency: a move is made, and it beats no move
    fast = dist.CommModel(us_per_unit=0.01, link_gbs=700.0, link_latency_us=5.0)
    pf = dist.place(c, None, 4, "skewed", B, 0.0, fast, rb)
    r = pf.residual
    assert r is not None and r.owner == 0 and r.split_row % 128 == 0
    m = B - r.split_row
    p = c[r.output] / B
    t = lambda rows: (fast.link_latency_us + rows * rb[r.output] / (1e3 * fast.link_gbs)) / fast.us_per_unit
    finish = max(L[0] - m * p, L[r.helper] + m * p + t(m))
    assert finish < L[0]
    # optimal within one 128-row tile: one tile more or less is not better
    for d in (-128, 128):
        m2 = m + d
        if 0 < m2 < B:
            assert finish <= max(L[0] - m2 * p, L[r.helper] + m2 * p + t(m2)) + 1e-9
    # the same imbalance over a link whose latency exceeds the whole gain: no move
    slow = dist.CommModel(us_per_unit=0.01, link_gbs=700.0, link_latency_us=0.01 * (L[0] - L.min()) * 1.01)
    assert dist.place(c, None, 4, "skewed", B, 0.0, slow, rb).residual is None
    # huge rows: the transfer outweighs the compute moved
    assert dist.place(c, None, 4, "skewed", B, 0.0, fast, [1e9] * 32).residual is None


def test_row_bytes_and_sparse_sources_c2():
    w = synth.c2_terabyte(0)
    nnz = np.full(26, 65536)
    rb = dist.row_bytes(w.spec, nnz, 65536)
    assert len(rb) == 34
    # a single-id table moves ~ offset + id in, length + offset + id out; a trigram 3 sources
    assert rb[0] == pytest.approx(4.125 + 8 + 12 + 8)
    assert rb[26] == pytest.approx(3 * 4.125 + 24 + 12 + 24)
    nodes = dist.sparse_output_nodes(w.spec)
    assert dist.sparse_sources(w.spec, nodes[26]) == [0, 1, 2]


def _slice_batch(h, r0, n):
    """Rows [r0, r0+n) of a host batch (r0 % 32 == 0); offsets stay absolute."""
    w0, w1 = r0 // 32, (r0 + n + 31) // 32
    return {"n_rows": n, "dense": [x[r0:r0 + n] for x in h["dense"]],
            "dense_valid": [None if v is None else v[w0:w1] for v in h["dense_valid"]],
            "sp_off": [o[r0:r0 + n + 1] for o in h["sp_off"]], "sp_val": h["sp_val"],
            "sp_valid": [None if v is None else v[w0:w1] for v in h["sp_valid"]]}


def _feature_lists(res, F, B):
    L, O, V = res["lengths"], res["offsets"], res["values"]
    return [[V[O[f * B + b]:O[f * B + b + 1]] for b in range(B)] for f in range(F)]


def _gloo_worker(rank, world, port, q):
    import torch
    import torch.distributed as tdist

    from oracle import oracle

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        w = synth.c2_terabyte(0)
        B = 1000
        h = synth.make_batch(w, B, seed=5)
        nodes = dist.sparse_output_nodes(w.spec)
        costs = np.ones(len(nodes))
        pl = dist.place(costs, dist.colocation(w.spec), world, "skewed", B, 0.05)
        res = pl.residual
        assert res is not None
        sub = dict(w.spec, outputs=[nodes[res.output]])
        n_hi = B - res.split_row
        # the piece each side sees has the same shapes: lengths, offsets, values (bound)
        bound = n_hi  # single-valued C2 lists: one id per row at most
        if rank == res.helper:
            hi = oracle.run(sub, _slice_batch(h, res.split_row, n_hi))
            vals = np.zeros(bound, np.int64)
            vals[: len(hi["values"])] = hi["values"]
            piece = [torch.from_numpy(hi["lengths"].astype(np.int32)), torch.from_numpy(hi["offsets"]),
                     torch.from_numpy(vals)]
            dist.nccl_exchange(rank, res, piece, None)
            q.put((rank, "sent"))
        elif rank == res.owner:
            bufs = [torch.zeros(n_hi, dtype=torch.int32), torch.zeros(n_hi + 1, dtype=torch.int64),
                    torch.zeros(bound, dtype=torch.int64)]
            dist.nccl_exchange(rank, res, None, bufs)
            lo = oracle.run(sub, _slice_batch(h, 0, res.split_row))
            # stitch exactly as rap_jagged_append does: T = running total
            T = int(lo["offsets"][-1])
            so = bufs[1].numpy()
            lengths = np.concatenate([lo["lengths"], bufs[0].numpy()])
            offsets = np.concatenate([lo["offsets"], T + so[1:] - so[0]])
            values = np.concatenate([lo["values"], bufs[2].numpy()[: int(so[-1] - so[0])]])
            full = oracle.run(sub, h)
            ok = (np.array_equal(lengths, full["lengths"]) and np.array_equal(offsets, full["offsets"])
                  and np.array_equal(values, full["values"]))
            q.put((rank, "ok" if ok else "MISMATCH"))
        else:
            q.put((rank, "idle"))
        tdist.barrier()
    finally:
        tdist.destroy_process_group()


def test_residual_exchange_gloo_world2():
    import torch.multiprocessing as mp

    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    got = dict(q.get(timeout=5) for _ in range(2))
    assert all(p.exitcode == 0 for p in procs), got
    assert sorted(got.values()) == ["ok", "sent"], got


# --------------------------------------------------- GPU: simulated ranks
@pytest.mark.gpu
@pytest.mark.parametrize("world,mode", [(2, "balanced"), (4, "round_robin"), (4, "skewed"), (8, "skewed")])
def test_sharded_ranks_match_oracle(world, mode):
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import rap
    from tests.parity import dense_close

    w = synth.c2_terabyte(0)
    B = 3000
    h = synth.make_batch(w, B, seed=21)
    raw = rap.DeviceBatch(h, "cuda:0")
    full = rap.Plan(w.spec, device=0)
    fo = rap.DeviceOutput(full, B, raw.sp_nnz, "cuda:0")
    full.preprocess(raw, fo)
    torch.cuda.synchronize()
    single = fo.to_numpy()
    want = oracle.run(w.spec, h)
    assert want["status"] == "OK"
    F = fo.f_out
    wl = _feature_lists(want, F, B)
    sl = _feature_lists(single, F, B)
    pl = dist.plan_placement(w.spec, B, raw.sp_nnz, world, mode, imbalance_tol=0.05)
    if mode == "skewed":
        assert pl.residual is not None
    ranks = [dist.ShardedPreprocessor(w.spec, pl, r, world, B, raw.sp_nnz, device=0) for r in range(world)]
    outs = [rk.new_output() for rk in ranks]
    box = {}

    def exchange(rank, res, piece, bufs):  # one-GPU stand-in for the NCCL send/recv
        if rank == res.helper:
            box["piece"] = [t.clone() for t in piece]
        elif rank == res.owner:
            for dst, src in zip(bufs, box["piece"]):
                dst.copy_(src)

    order = list(range(world))
    if pl.residual is not None:  # the helper's piece exists before the owner stitches
        order.remove(pl.residual.helper)
        order.insert(0, pl.residual.helper)
    for r in order:
        ranks[r].preprocess(raw, outs[r], exchange=exchange)
    torch.cuda.synchronize()
    seen = []
    for r in range(world):
        got = outs[r].to_numpy()
        r0, n = dist.shard_rows(B, r, world)
        assert dense_close(got["dense"], want["dense"][r0:r0 + n]).all(), r
        assert np.array_equal(got["dense"].view(np.uint32), single["dense"][r0:r0 + n].view(np.uint32))
        gl = _feature_lists(got, len(got["features"]), B)
        for k, j in enumerate(got["features"]):
            assert all(np.array_equal(a, b) for a, b in zip(gl[k], wl[j])), (r, j)
            assert all(np.array_equal(a, b) for a, b in zip(gl[k], sl[j])), (r, j)
        L = got["lengths"].reshape(-1)
        assert got["offsets"][0] == 0 and np.array_equal(np.diff(got["offsets"]), L)
        seen += got["features"]
    assert sorted(seen) == list(range(F))
    for rk in ranks:
        rk.close()
    full.close()


# ------------------------------------------- GPU: two processes, one device
def _gpu_rank_worker(rank, world, port, mode, q):
    import torch
    import torch.distributed as tdist

    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import rap
    from tests.parity import dense_close

    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        tdist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        w = synth.c2_terabyte(0)
        B = 2600
        h = synth.make_batch(w, B, seed=33)
        sp_nnz = np.array([int(o[-1]) - int(o[0]) for o in h["sp_off"]], dtype=np.int64)
        pl = dist.plan_placement(w.spec, B, sp_nnz, world, mode, imbalance_tol=0.05)
        sp = dist.ShardedPreprocessor(w.spec, pl, rank, world, B, sp_nnz, device=0)
        # this rank uploads only its own tables' columns and its dense shard
        raw = rap.DeviceBatch(h, "cuda:0", sparse_cols=sp.sparse_columns(), dense_rows=(sp.row0, sp.dense_rows))
        full = rap.DeviceBatch(h, "cuda:0")
        assert raw.uploaded_bytes() < full.uploaded_bytes()
        del full
        out = sp.new_output()
        for _ in range(2):  # twice: the chained launch and the append are re-entrant
            sp.preprocess(raw, out, exchange=dist.gloo_exchange)
        torch.cuda.synchronize()
        got = out.to_numpy()
        want = oracle.run(w.spec, h)
        F = len(dist.sparse_output_nodes(w.spec))
        wl = _feature_lists(want, F, B)
        gl = _feature_lists(got, len(got["features"]), B)
        assert dense_close(got["dense"], want["dense"][sp.row0:sp.row0 + sp.dense_rows]).all()
        for k, j in enumerate(got["features"]):
            assert all(np.array_equal(a, b) for a, b in zip(gl[k], wl[j])), (rank, j)
        assert got["offsets"][0] == 0 and np.array_equal(np.diff(got["offsets"]), got["lengths"].reshape(-1))
        res = pl.residual
        q.put((rank, {"features": got["features"], "residual": None if res is None else res.__dict__}))
        sp.close()
        tdist.destroy_process_group()
    except Exception as e:  # noqa: BLE001 - reported to the parent
        import traceback

        q.put((rank, "ERR " + repr(e) + traceback.format_exc()[-1500:]))


@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["skewed", "balanced"])
def test_two_processes_one_gpu_vs_oracle(mode):
    """Two ranks as two processes on one B200 (gloo group, host-staged
    residual exchange): each uploads only its own columns and dense shard, and
    its KJT features and dense rows equal the oracle's single-process result."""
    import multiprocessing as mp

    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gpu_rank_worker, args=(r, 2, port, mode, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=600) for _ in range(2))
    for p in procs:
        p.join(120)
    errs = {r: got[r] for r in range(2) if isinstance(got[r], str)}
    assert not errs, errs
    assert all(p.exitcode == 0 for p in procs)
    feats = sorted(got[0]["features"] + got[1]["features"])
    assert feats == list(range(34))
    if mode == "skewed":
        assert got[0]["residual"] is not None


# ---- joint mapping loop (rap_place_joint, §7.2) ----
def _joint_times(costs, colocate, home, owner, world, n_rows, cm, row_bytes):
    """Independent restatement of rap_place_joint's cost model: a graph runs
    on its owner (compute + its exchange when away from home), a duplicated
    graph (owner -1) on every rank."""
    T = [0.0] * world
    for j, c in enumerate(costs):
        us = c * cm.us_per_unit
        if owner[j] < 0:
            for r in range(world):
                T[r] += us
            continue
        T[owner[j]] += us
        if owner[j] != home[j]:
            # exchange charged once per colocated group (at its anchor)
            anchor = j
            while colocate is not None and colocate[anchor] >= 0:
                anchor = colocate[anchor]
            grp = [k for k in range(len(costs)) if _anchor(colocate, k) == anchor]
            if j == anchor:
                T[owner[j]] += cm.link_latency_us + sum(n_rows * row_bytes[k] / (1e3 * cm.link_gbs) for k in grp)
    return T


def _anchor(colocate, k):
    while colocate is not None and colocate[k] >= 0:
        k = colocate[k]
    return k


def test_joint_mapping_keeps_locality_when_moves_do_not_pay():
    costs = [100.0] * 8 + [300.0] * 8
    home = [0] * 8 + [1] * 8
    slow = dist.CommModel(us_per_unit=0.01, link_gbs=0.001, link_latency_us=1e6)
    m = dist.place_joint(costs, None, home, 2, 65536, slow, [100.0] * 16)
    assert m.owner == home and m.moves == 0


def test_joint_mapping_balances_a_skewed_home_and_stops_at_a_local_optimum():
    rng = np.random.default_rng(7)
    n, world, B = 40, 4, 65536
    costs = list(rng.uniform(50, 500, n))
    home = [0 if j < n // 2 else 1 + j % (world - 1) for j in range(n)]  # rank 0: half the graphs (skew)
    rb = list(rng.uniform(8, 40, n))
    cm = dist.CommModel(us_per_unit=0.02, link_gbs=700.0, link_latency_us=5.0)
    m = dist.place_joint(costs, None, home, world, B, cm, rb)
    T0 = _joint_times(costs, None, home, home, world, B, cm, rb)
    T = _joint_times(costs, None, home, m.owner, world, B, cm, rb)
    assert np.allclose(T, m.times, rtol=1e-9)
    assert m.moves > 0 and max(T) < max(T0)
    # stopping rule: no single graph of the costliest rank lowers the cost on the cheapest one
    h, lo = int(np.argmax(T)), int(np.argmin(T))
    for j in range(n):
        if m.owner[j] != h:
            continue
        o = list(m.owner)
        o[j] = lo
        assert max(_joint_times(costs, None, home, o, world, B, cm, rb)) >= max(T) - 1e-9


def test_joint_mapping_duplicated_and_colocated_graphs():
    costs = [200.0, 50.0, 400.0, 100.0, 30.0]
    colocate = [-1, 0, -1, -1, -1]  # output 1 (an NGram) shares output 0's rank
    home = [0, 0, 0, -1, 0]         # output 3: a row-wise table, duplicated on every rank
    cm = dist.CommModel(us_per_unit=0.05, link_gbs=700.0, link_latency_us=1.0)
    m = dist.place_joint(costs, colocate, home, 3, 4096, cm, [16.0] * 5)
    assert m.owner[3] == -1
    assert m.owner[0] == m.owner[1]
    T = _joint_times(costs, colocate, home, m.owner, 3, 4096, cm, [16.0] * 5)
    assert np.allclose(T, m.times, rtol=1e-9)
    assert all(t >= 100.0 * 0.05 for t in T)  # the duplicated graph's compute on every rank


def test_joint_mapping_rejects_bad_input():
    cm = dist.CommModel(us_per_unit=0.05)
    with pytest.raises(rap.RapError):
        dist.place_joint([1.0, 2.0], [-1, 0], [0, 1], 2, 128, cm, [1.0, 1.0])  # colocated, different homes
    with pytest.raises(rap.RapError):
        dist.place_joint([1.0], None, [5], 2, 128, cm, [1.0])  # home out of range
