"""Parity of the CUDA path (through the C ABI) against the CPU oracle.

Integer outputs bit-exact, dense f32 within the R16 rule (tests/parity.py).
Sizes span several descriptors (1024 sparse rows, 128 dense rows each) and a
ragged tail; the full-size C1 / C2 configurations are compared completely.
"""
import numpy as np
import pytest

from tests.helpers import batch, dense_from_values, node, sparse_from_lists, spec
from tests.parity import assert_parity

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth
    from oracle import oracle

    rap.load()
    return rap, synth, oracle, torch


@pytest.fixture(params=[1, 2, 3], ids=["tiled", "rows", "jit"], autouse=True)
def kernel_mode(request):
    """Every parity case runs on every fused kernel (rap_set_kernel): tiled,
    interpreted row-block and the plan-specialised (generated) row-block kernel."""
    from paper_conf_asplos_wangwdz0d24_b200 import rap

    old = rap.DEFAULT_KERNEL
    rap.DEFAULT_KERNEL = request.param
    yield request.param
    rap.DEFAULT_KERNEL = old


def run_gpu(rap, torch, spec_, host, budget=0, plan=None, dense_ld=None):
    own = plan is None
    if own:
        plan = rap.Plan(spec_, device=0, sm_budget=budget)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, host["n_rows"], raw.sp_nnz, "cuda:0", dense_ld=dense_ld)
    plan.preprocess(raw, out)
    torch.cuda.synchronize()
    got = out.to_numpy()
    if own:
        plan.close()
    return got


def check(env, spec_, host, **kw):
    rap, synth, oracle, torch = env
    want = oracle.run(spec_, host)
    got = run_gpu(rap, torch, spec_, host, **kw)
    assert_parity(got, want)
    return got, want


# ------------------------------------------------------------------ configurations
@pytest.mark.parametrize("B", [1, 31, 1000, 4096, 5000])
def test_c1_kaggle(env, B):
    _, synth, _, _ = env
    w = synth.c1_kaggle(0)
    check(env, w.spec, synth.make_batch(w, B, seed=B))


@pytest.mark.parametrize("B", [1, 129, 3000, 9999])
def test_c2_terabyte_ragged(env, B):
    _, synth, _, _ = env
    w = synth.c2_terabyte(0)
    check(env, w.spec, synth.make_batch(w, B, seed=B + 7))


@pytest.mark.parametrize("n_ngram,B", [(64, 1000), (128, 4099)])
def test_c2_many_ngram_outputs(env, n_ngram, B):
    """The growing-NGram graphs (Fig 11 sweep): 90 / 154 sparse outputs, past
    an interpreted group's 64 -- the generated kernel takes them as one group
    (kJitMaxF), the others split groups."""
    _, synth, _, _ = env
    w = synth.c2_terabyte(0, n_ngram=n_ngram)
    check(env, w.spec, synth.make_batch(w, B, seed=B + n_ngram))


def test_c2_terabyte_full_size(env):
    """BASELINE config 2 at its full batch (65536), the launch bench.py times."""
    _, synth, _, _ = env
    w = synth.c2_terabyte(0)
    got, want = check(env, w.spec, synth.make_batch(w, 65536, seed=1))
    assert got["values"].shape[0] == 34 * 65536


def test_single_output_plans(env):
    """Every output of the C2 graph as its own plan (the unfused arm of bench.py's
    fusion ablation): dense-only and sparse-only plans, each equal to the oracle."""
    _, synth, _, _ = env
    w = synth.c2_terabyte(0)
    host = synth.make_batch(w, 1500, seed=5)
    rap, _, oracle, torch = env
    for i, o in enumerate(w.spec["outputs"]):
        s = dict(w.spec)
        s["outputs"] = [o]
        assert_parity(run_gpu(rap, torch, s, host), oracle.run(s, host), ctx=f"output {i} (node {o})")
    # dense-only plan through the host-buffer entry: offsets = [0]
    s = dict(w.spec)
    s["outputs"] = [w.spec["outputs"][0]]
    plan = rap.Plan(s, device=0)
    hraw = rap.DeviceBatch(host, None, pin=True)
    hout = rap.DeviceOutput(plan, host["n_rows"], hraw.sp_nnz, None, pin=True)
    hout.offsets.fill_(-7)
    plan.preprocess_host(hraw, hout)
    assert_parity(hout.to_numpy(), oracle.run(s, host), ctx="dense-only host entry")
    plan.close()


def test_multihot_small(env):
    _, synth, _, _ = env
    w = synth.c4_multihot(0, n_features=24)
    check(env, w.spec, synth.make_batch(w, 2500, seed=3))


# ------------------------------------------------------------------ edge cases
def test_empty_batch(env):
    rap, synth, oracle, torch = env
    w = synth.c2_terabyte(0)
    host = synth.make_batch(w, 0, seed=1)
    got = run_gpu(rap, torch, w.spec, host)
    assert list(got["offsets"]) == [0]
    assert got["values"].size == 0


def test_unaligned_offsets_null_segments_no_bitmaps(env):
    _, synth, _, _ = env
    w = synth.c2_terabyte(0)
    check(env, w.spec, synth.make_batch(w, 2100, seed=5, null_segments=True, base_offset=3))
    check(env, w.spec, synth.make_batch(w, 2100, seed=6, drop_bitmaps=True))


def test_all_null_and_all_empty(env):
    rows_null = [None] * 1500
    rows_empty = [[] for _ in range(1500)]
    d = dense_from_values([None] * 1500)
    s = spec(1, 2, [node("fillnull", [("s", 0)], i_fill=4), node("firstx", [("n", 0)], x=3),
                    node("sigridhash", [("s", 1)], salt=3, max_value=100),
                    node("ngram", [("s", 0), ("s", 1)], n=1, salt=2, max_value=50),
                    node("logit", [("d", 0)], eps=1e-6), node("fillnull", [("d", 0)], f_fill=2.5)],
             [1, 2, 3, 4, 5])
    check(env, s, batch(1500, dense=[d], sparse=[sparse_from_lists(rows_null), sparse_from_lists(rows_empty)]))


def test_huge_list_and_firstx(env):
    rng = np.random.default_rng(0)
    rows = [list(rng.integers(0, 2**40, 3)) for _ in range(700)]
    rows[333] = list(rng.integers(0, 2**40, 1_000_000))
    sp = sparse_from_lists(rows)
    s = spec(0, 1, [node("sigridhash", [("s", 0)], salt=9, max_value=10**9),
                    node("firstx", [("n", 0)], x=5),
                    node("clamp", [("s", 0)], lo=10, hi=2**39)],
             [0, 1, 2])
    check(env, s, batch(700, sparse=[sp]))


def test_straddling_lists_and_long_rows(env):
    """Lists of 0..200 ids so row groups straddle warps / descriptors."""
    rng = np.random.default_rng(1)
    rows = [None if rng.random() < 0.1 else list(rng.integers(-5, 2**33, rng.integers(0, 200))) for _ in range(3100)]
    sp = sparse_from_lists(rows, base_offset=11)
    s = spec(0, 1, [node("fillnull", [("s", 0)], i_fill=-1),
                    node("clamp", [("n", 0)], lo=0, hi=2**32),
                    node("sigridhash", [("n", 1)], salt=77, max_value=123457),
                    node("firstx", [("n", 2)], x=150),
                    node("ngram", [("n", 3)], n=4, salt=5, max_value=10**7),
                    node("onehot", [("s", 0)], k=40)],
             [3, 4, 5])
    check(env, s, batch(3100, sparse=[sp]))


def test_dense_edge_values(env):
    vals = [0.0, 1.0, 0.5, 1e-7, 1 - 1e-7, -1.0, 2.0, float("nan"), float("inf"), -float("inf"), None, 1e30,
            1e-30, 3.0, 4.0, 1.0001, 0.9999] * 90
    d = dense_from_values(vals)
    nodes = [node("logit", [("d", 0)], eps=1e-6), node("logit", [("d", 0)], eps=0.25)]
    for lam in (0.0, 0.25, 0.5, -0.5, 1.0, -1.0, 2.0):
        nodes.append(node("boxcox", [("d", 0)], **{"lambda": lam}))
    nodes.append(node("fillnull", [("d", 0)], f_fill=-3.0))
    nodes.append(node("bucketize", [("d", 0)], borders=np.array([-1.0, 0.0, 0.5, 1.0, 1.0, 3.0], dtype=np.float32)))
    nodes.append(node("onehot", [("n", len(nodes) - 1)], k=7))
    nodes.append(node("bucketize", [("n", len(nodes) - 3)], borders=np.array([0.0, 2.0], dtype=np.float32)))
    outs = list(range(len(nodes)))
    outs.remove(len(nodes) - 3)  # bucketize node -> used through onehot; keep the second bucketize as sparse out
    check(env, spec(1, 0, nodes, outs), batch(len(vals), dense=[d]))


def test_dense_ld_padding(env):
    _, synth, _, _ = env
    w = synth.c2_terabyte(0)
    check(env, w.spec, synth.make_batch(w, 777, seed=2), dense_ld=53)


# ------------------------------------------------------------------ metamorphic / scheduling
def test_budget_invariance_and_repeat(env):
    rap, synth, oracle, torch = env
    w = synth.c2_terabyte(0)
    host = synth.make_batch(w, 20000, seed=4)
    want = oracle.run(w.spec, host)
    plan = rap.Plan(w.spec, device=0)
    for budget in (1, 3, 17, 0, 148):
        plan.set_budget(min(budget, plan.info()["sm_count"]))
        for _ in range(2):
            assert_parity(run_gpu(rap, torch, w.spec, host, plan=plan), want, f"budget {budget}")
    # different n_rows on the same plan (descriptor table re-upload, scan-state growth)
    for B in (5, 40000, 1024, 1025):
        h2 = synth.make_batch(w, B, seed=B)
        assert_parity(run_gpu(rap, torch, w.spec, h2, plan=plan), oracle.run(w.spec, h2), f"B={B}")
    plan.close()


def test_many_launches_same_plan(env):
    """Ticket / done counters and the look-back epoch are reset on the device."""
    rap, synth, oracle, torch = env
    w = synth.c1_kaggle(0)
    host = synth.make_batch(w, 4096, seed=9)
    want = oracle.run(w.spec, host)
    plan = rap.Plan(w.spec, device=0)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, 4096, raw.sp_nnz, "cuda:0")
    for _ in range(300):
        plan.preprocess(raw, out)
    torch.cuda.synchronize()
    assert_parity(out.to_numpy(), want)
    plan.close()


def test_partition_cache_across_batch_shapes(env):
    """One plan over 12 batches whose null rates / list lengths differ (cached,
    near-shape-reused and evicted work partitions): every output exact."""
    rap, synth, oracle, torch = env
    w = synth.c4_multihot(0, n_features=16)
    plan = rap.Plan(w.spec, device=0)
    for i in range(12):
        host = synth.make_batch(w, 1024 + 128 * (i % 10), seed=40 + i)
        got = run_gpu(rap, torch, w.spec, host, plan=plan)
        assert_parity(got, oracle.run(w.spec, host), ctx=f"batch {i}")
    plan.close()


def test_cuda_graph_replay(env):
    rap, synth, oracle, torch = env
    w = synth.c2_terabyte(0)
    host = synth.make_batch(w, 6000, seed=12)
    want = oracle.run(w.spec, host)
    plan = rap.Plan(w.spec, device=0)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, 6000, raw.sp_nnz, "cuda:0")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        plan.preprocess(raw, out, stream=s)  # warm-up: descriptor table + scan state
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        plan.preprocess(raw, out, stream=s)
    for _ in range(5):
        out.values.fill_(-1)
        g.replay()
    torch.cuda.synchronize()
    assert_parity(out.to_numpy(), want)
    plan.close()


def test_host_buffers_entry(env):
    rap, synth, oracle, torch = env
    w = synth.c2_terabyte(0)
    host = synth.make_batch(w, 5000, seed=21, base_offset=2)
    want = oracle.run(w.spec, host)
    plan = rap.Plan(w.spec, device=0)
    raw = rap.DeviceBatch(host, None, pin=True)
    out = rap.DeviceOutput(plan, 5000, raw.sp_nnz, None, pin=True)
    for _ in range(2):
        plan.preprocess_host(raw, out)
    assert_parity(out.to_numpy(), want)
    plan.close()


def test_host_entry_gather_alignments(env):
    """The host entry's batched H2D (one gather launch over pinned columns):
    sources only 8- / 4-byte aligned (an odd first offset, a ragged offsets
    array) and columns smaller than one chunk; pageable columns take the
    per-column copies.  Every case equal to the oracle."""
    rap, synth, oracle, torch = env
    w = synth.c2_terabyte(0)
    for B, base, where in ((4101, 3, None), (37, 5, None), (70001, 1, None), (1500, 3, "cpu")):
        host = synth.make_batch(w, B, seed=B, base_offset=base)
        plan = rap.Plan(w.spec, device=0)
        raw = rap.DeviceBatch(host, where, pin=where is None)
        out = rap.DeviceOutput(plan, B, raw.sp_nnz, None, pin=True)
        plan.preprocess_host(raw, out)
        assert_parity(out.to_numpy(), oracle.run(w.spec, host), ctx=f"B={B} base={base} {where or 'pinned'}")
        plan.close()


def test_host_async_two_plans_pipelined(env):
    """rap_preprocess_host_async: two plans on two streams, batches alternating,
    each result equal to the oracle once its stream is synchronised."""
    rap, synth, oracle, torch = env
    w = synth.c2_terabyte(0)
    hosts = [synth.make_batch(w, 3000 + 100 * i, seed=40 + i) for i in range(4)]
    plans = [rap.Plan(w.spec, device=0), rap.Plan(w.spec, device=0)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    raws = [rap.DeviceBatch(h, None, pin=True) for h in hosts]
    outs = [rap.DeviceOutput(plans[i % 2], h["n_rows"], raws[i].sp_nnz, None, pin=True) for i, h in enumerate(hosts)]
    for i in range(4):
        plans[i % 2].preprocess_host_async(raws[i], outs[i], streams[i % 2])
    torch.cuda.synchronize()
    for i in range(4):
        assert_parity(outs[i].to_numpy(), oracle.run(w.spec, hosts[i]), ctx=f"batch {i}")
    for p_ in plans:
        p_.close()


def test_capacity_error(env):
    rap, synth, oracle, torch = env
    w = synth.c1_kaggle(0)
    host = synth.make_batch(w, 100, seed=1)
    plan = rap.Plan(w.spec, device=0)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, 100, raw.sp_nnz, "cuda:0", capacity=10)
    with pytest.raises(rap.RapError) as ei:
        plan.preprocess(raw, out)
    assert ei.value.status == "CAPACITY"
    plan.close()


# ------------------------------------------------------------------ random graphs
def _random_graph(rng, n_dense, n_sparse):
    nodes, outs = [], []

    def add(op, inputs, **kw):
        nodes.append(node(op, inputs, **kw))
        return ("n", len(nodes) - 1)

    def id_chain(src, depth):
        cur = src
        for _ in range(depth):
            k = rng.integers(0, 6)
            if k == 0:
                cur = add("fillnull", [cur], i_fill=int(rng.integers(-3, 3)))
            elif k == 1:
                cur = add("clamp", [cur], lo=int(rng.integers(-10, 0)), hi=int(rng.integers(0, 2**34)))
            elif k == 2:
                cur = add("sigridhash", [cur], salt=int(rng.integers(0, 2**63)), max_value=int(rng.integers(1, 10**8)))
            elif k == 3:
                b = np.sort(rng.integers(-100, 2**33, int(rng.integers(1, 300)))).astype(np.int64)
                cur = add("bucketize", [cur], borders=b)
            elif k == 4:
                cur = add("firstx", [cur], x=int(rng.integers(0, 6)))
            else:
                keys = rng.choice(np.arange(-20, 2000), int(rng.integers(0, 50)), replace=False).astype(np.int64)
                cur = add("mapid", [cur], keys=keys, vals=rng.integers(-5, 10**6, len(keys)),
                          map_default=int(rng.integers(-9, 9)))
        return cur

    def dense_chain(c, depth):
        cur = ("d", c)
        for _ in range(depth):
            k = rng.integers(0, 3)
            if k == 0:
                cur = add("fillnull", [cur], f_fill=float(rng.uniform(-1, 2)))
            elif k == 1:
                cur = add("logit", [cur], eps=float(rng.choice([1e-6, 1e-3, 0.1])))
            else:
                cur = add("boxcox", [cur], **{"lambda": float(rng.choice([0.0, 0.25, 0.5, -0.5, 1.5]))})
        return cur

    for c in range(n_dense):
        outs.append(dense_chain(c, int(rng.integers(1, 4)))[1])
    chains = []
    for s in range(n_sparse):
        ch = id_chain(("s", s), int(rng.integers(1, 5)))
        chains.append(ch)
        outs.append(ch[1])
    # dense -> bucketize -> id chain as a sparse output
    db = add("bucketize", [dense_chain(0, 1)], borders=np.sort(rng.uniform(-2, 2, 9)).astype(np.float32))
    outs.append(id_chain(db, 2)[1])
    chains.append(db)
    # NGram over 1..3 chains, with post ops
    for _ in range(3):
        k = int(rng.integers(1, 4))
        srcs = [chains[int(i)] for i in rng.choice(len(chains), k, replace=False)]
        ng = add("ngram", srcs, n=int(rng.integers(1, 5)), salt=int(rng.integers(0, 2**60)),
                 max_value=int(rng.integers(1, 10**9)))
        outs.append(id_chain(ng, int(rng.integers(0, 3)))[1] if rng.random() < 0.5 else ng[1])
    # OneHot over a sparse chain and over an NGram
    outs.append(add("onehot", [chains[0]], k=int(rng.integers(1, 90)))[1])
    outs.append(add("onehot", [("n", outs[-2])], k=70)[1])
    return {"n_dense": n_dense, "n_sparse": n_sparse, "nodes": nodes, "outputs": outs}


@pytest.mark.parametrize("seed", range(6))
def test_random_graphs(env, seed):
    _, synth, _, _ = env
    rng = np.random.default_rng(100 + seed)
    n_dense, n_sparse = 3, 4
    s = _random_graph(rng, n_dense, n_sparse)
    B = int(rng.integers(500, 4000))
    dense = [synth.dense_column(seed, c, "unit" if c % 2 else "count", B) for c in range(n_dense)]
    means = [None, 3.0, 0.5, 12.0]
    sparse = [synth.sparse_column(seed, sc, 5000, B, means[sc], null_p=0.15, null_segments=(sc == 2),
                                  base_offset=sc) for sc in range(n_sparse)]
    check(env, s, batch(B, dense=dense, sparse=sparse))


@pytest.mark.parametrize("plan_id", [2, 3])
def test_table3_plan_graphs(env, plan_id, kernel_mode):
    """Table 3 Plan 2 (26 dense / 52 sparse features, 384 ops) and Plan 3
    (52 / 104, 1548 ops) shaped graphs (synth.plan_graph): deep non-canonical
    chains, hundreds of NGram outputs, > 64 raw sparse columns (Plan 3: the
    tiled kernel's large template only), ragged batch."""
    _, synth, _, _ = env
    if plan_id == 3 and kernel_mode != 1:
        pytest.skip("Plan 3 reads 104 raw sparse columns: the row-block kernels take <= 64")
    w = synth.plan_graph(plan_id, 0)
    check(env, w.spec, synth.make_batch(w, 1111, seed=plan_id))
