"""Edge-case parity of every fused kernel against the CPU oracle (VERDICT r01
"parity holes"): table sizes M >= 2^32 (the 64x64 multiply-high reduction),
a MapId table holding INT64_MIN, NGram over k = 5..8 sources, programs longer
than the 32 ops an SProg stages and dense groups beyond 96 ops, Clamp and ids
at INT64_MIN / INT64_MAX, and the device-side capacity-overflow flag
(rap_check_overflow).  Integer outputs bit-exact, dense within R16
(tests/parity.py).  PAPER.md Table 1 (L440-463); readings DESIGN.md §3.
"""
import numpy as np
import pytest

from tests.helpers import batch, dense_from_values, node, sparse_from_lists, spec
from tests.parity import assert_parity

pytestmark = pytest.mark.gpu

I64_MIN, I64_MAX = -(2**63), 2**63 - 1


@pytest.fixture(scope="module")
def env():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth
    from oracle import oracle

    rap.load()
    return rap, synth, oracle, torch


@pytest.fixture(params=[1, 2, 3], ids=["tiled", "rows", "jit"])
def kmode(request):
    return request.param


def run_check(env, kmode, s, host, ctx=""):
    rap, synth, oracle, torch = env
    want = oracle.run(s, host)
    plan = rap.Plan(s, device=0)
    plan.set_kernel(kmode)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, host["n_rows"], raw.sp_nnz, "cuda:0")
    plan.preprocess(raw, out)
    torch.cuda.synchronize()
    got = out.to_numpy()
    assert plan.check_overflow() == 0
    plan.close()
    assert_parity(got, want, ctx)
    return got


def _lists(rng, n, lo, hi, max_len=3, p_null=0.1, extremes=()):
    rows = []
    for _ in range(n):
        if rng.random() < p_null:
            rows.append(None)
            continue
        k = int(rng.integers(0, max_len + 1))
        rows.append([int(v) for v in rng.integers(lo, hi, k)])
    for i, e in enumerate(extremes):  # pin a few rows to the extremes
        rows[(7 * i + 3) % n] = [e]
    return rows


def test_large_M_sigrid_and_ngram(env, kmode):
    """M = 2^32, 2^40, 2^63 - 1: the reduction floor(h * M / 2^64) on the
    __umul64hi path (R2), for SigridHash and for NGram windows (R3, R7)."""
    rng = np.random.default_rng(1)
    B = 1500
    sp = [sparse_from_lists(_lists(rng, B, -(2**40), 2**40, extremes=(I64_MIN, I64_MAX, 0, -1)))
          for _ in range(2)]
    nodes, outs = [], []
    for k, M in enumerate((2**32, 2**40, 2**63 - 1)):
        nodes.append(node("sigridhash", [("s", 0)], salt=11 + k, max_value=M))
        outs.append(len(nodes) - 1)
        nodes.append(node("ngram", [("s", 0), ("s", 1)], n=2, salt=5 + k, max_value=M))
        outs.append(len(nodes) - 1)
    nodes.append(node("fillnull", [("s", 1)], i_fill=I64_MIN))
    nodes.append(node("sigridhash", [("n", len(nodes) - 1)], salt=3, max_value=2**63 - 1))
    outs.append(len(nodes) - 1)
    run_check(env, kmode, spec(0, 2, nodes, outs), batch(B, sparse=sp))


def test_mapid_int64_min_key_and_clamp_extremes(env, kmode):
    """A MapId table holding INT64_MIN (the interpreter's has_min path, R8) and
    Clamp at the int64 extremes (identity bounds and pinned bounds, R6)."""
    rng = np.random.default_rng(2)
    B = 1300
    rows = _lists(rng, B, -50, 50, extremes=(I64_MIN, I64_MAX, I64_MIN, 0))
    sp = sparse_from_lists(rows)
    keys = np.array([I64_MIN, 0, 5, -7, I64_MAX, 42], dtype=np.int64)
    vals = np.array([111, 222, 333, 444, 555, I64_MIN], dtype=np.int64)
    nodes = [node("mapid", [("s", 0)], keys=keys, vals=vals, map_default=-9),
             node("clamp", [("s", 0)], lo=I64_MIN, hi=I64_MAX),
             node("clamp", [("s", 0)], lo=I64_MIN, hi=I64_MIN),
             node("clamp", [("s", 0)], lo=I64_MAX, hi=I64_MAX),
             node("clamp", [("s", 0)], lo=-3, hi=I64_MAX),
             node("fillnull", [("s", 0)], i_fill=I64_MAX),
             node("mapid", [("n", 5)], keys=keys, vals=vals, map_default=I64_MIN),
             node("sigridhash", [("n", 6)], salt=I64_MAX, max_value=2**40)]
    run_check(env, kmode, spec(0, 1, nodes, [0, 1, 2, 3, 4, 6, 7]), batch(B, sparse=[sp]))


@pytest.mark.parametrize("k", [5, 6, 7, 8])
def test_ngram_many_sources(env, kmode, k):
    """NGram over k = 5..8 source lists (R7: concatenation in source order),
    windows n in {2, k} so rows with several windows and exactly one occur."""
    rng = np.random.default_rng(10 + k)
    B = 900
    sp = [sparse_from_lists(_lists(rng, B, 0, 10**6, max_len=2, p_null=0.2)) for _ in range(k)]
    nodes = [node("fillnull", [("s", i)], i_fill=i) for i in range(k)]
    nodes.append(node("ngram", [("n", i) for i in range(k)], n=2, salt=9, max_value=10**7))
    nodes.append(node("ngram", [("s", i) for i in range(k)], n=k, salt=8, max_value=2**35))
    nodes.append(node("firstx", [("n", k)], x=3))
    run_check(env, kmode, spec(0, k, nodes, [k, k + 1, k + 2]), batch(B, sparse=sp))


def test_long_programs(env, kmode):
    """An id chain of 40 ops (beyond the 32 an SProg stages: global op indices)
    and a dense group of 120 ops (beyond the 96 a DProg stages)."""
    rng = np.random.default_rng(3)
    B = 1100
    sp = sparse_from_lists(_lists(rng, B, -(2**33), 2**33, max_len=4))
    nodes, cur = [], ("s", 0)
    for i in range(40):
        if i % 3 == 0:
            nodes.append(node("clamp", [cur], lo=-(2**34) + i, hi=2**34 - i))
        elif i % 3 == 1:
            nodes.append(node("sigridhash", [cur], salt=i, max_value=2**31 + i))
        else:
            nodes.append(node("mapid", [cur], keys=np.arange(i, i + 40, dtype=np.int64),
                              vals=np.arange(40, dtype=np.int64) * 3, map_default=-i))
        cur = ("n", len(nodes) - 1)
    outs = [len(nodes) - 1]
    vals = [0.1, 0.5, 0.9, None, float("nan"), 2.0, 0.0, 1.0] * (B // 8 + 1)
    d = dense_from_values(vals[:B])
    for c in range(30):  # 30 dense outputs x (FillNull, Logit, BoxCox, FillNull) = 120 ops over the groups
        nodes.append(node("fillnull", [("d", 0)], f_fill=0.25 + 0.01 * c))
        nodes.append(node("logit", [("n", len(nodes) - 1)], eps=1e-6 * (c + 1)))
        nodes.append(node("boxcox", [("n", len(nodes) - 1)], **{"lambda": 0.5}))
        nodes.append(node("fillnull", [("n", len(nodes) - 1)], f_fill=-1.0))
        outs.append(len(nodes) - 1)
    # one dense chain of 101 ops (more than a DProg carries: global op indices)
    cur = ("d", 0)
    for i in range(100):
        nodes.append(node("fillnull", [cur], f_fill=0.125 * (i % 5)))
        cur = ("n", len(nodes) - 1)
    nodes.append(node("logit", [cur], eps=1e-3))
    outs.append(len(nodes) - 1)
    run_check(env, kmode, spec(1, 1, nodes, outs), batch(B, dense=[d], sparse=[sp]))


def test_capacity_overflow_flag(env, kmode):
    """sp_nnz understating the batch: values past values_capacity are not
    written and rap_check_overflow reports it (then clears it)."""
    rap, synth, oracle, torch = env
    w = synth.c1_kaggle(0)
    host = synth.make_batch(w, 3000, seed=2)
    plan = rap.Plan(w.spec, device=0)
    plan.set_kernel(kmode)
    raw = rap.DeviceBatch(host, "cuda:0")
    small = np.zeros_like(raw.sp_nnz)  # claims empty columns: bound = 0 ids
    raw.sp_nnz[:] = small
    out = rap.DeviceOutput(plan, 3000, raw.sp_nnz, "cuda:0", capacity=100)
    plan.preprocess(raw, out)
    torch.cuda.synchronize()
    assert plan.check_overflow() == 1
    assert plan.check_overflow() == 0  # cleared
    plan.close()


def test_plans_with_different_smem_interleave(env, kmode):
    """plan A (a 300-wide OneHot group: large dynamic smem) is
    launched, plan B (small smem) is created and launched, then A launches
    again -- the kernels' MaxDynamicSharedMemorySize must still admit A."""
    rap, synth, oracle, torch = env
    rng = np.random.default_rng(4)
    B = 700
    sp = sparse_from_lists(_lists(rng, B, 0, 300, max_len=2))
    wide = spec(0, 1, [node("onehot", [("s", 0)], k=300), node("sigridhash", [("s", 0)], salt=1, max_value=1000)],
                [0, 1])
    host = batch(B, sparse=[sp])
    want_a = oracle.run(wide, host)
    w = synth.c1_kaggle(0)
    hb = synth.make_batch(w, 500, seed=9)
    want_b = oracle.run(w.spec, hb)

    def launch(plan, h):
        raw = rap.DeviceBatch(h, "cuda:0")
        out = rap.DeviceOutput(plan, h["n_rows"], raw.sp_nnz, "cuda:0")
        plan.preprocess(raw, out)
        torch.cuda.synchronize()
        return out.to_numpy()

    a = rap.Plan(wide, device=0)
    a.set_kernel(kmode)
    assert_parity(launch(a, host), want_a, "A first")
    b = rap.Plan(w.spec, device=0)
    b.set_kernel(kmode)
    assert_parity(launch(b, hb), want_b, "B")
    assert_parity(launch(a, host), want_a, "A after B")
    c = rap.Plan(w.spec, device=0)  # another small plan created between launches
    assert_parity(launch(a, host), want_a, "A after C created")
    for p in (a, b, c):
        p.close()


def _exact_nnz_lists(B, nnz, seed):
    """B lists with exactly nnz ids (lengths 0..2*nnz/B), no nulls."""
    rng = np.random.default_rng(seed)
    lens = np.full(B, nnz // B)
    lens[: nnz - lens.sum()] += 1
    rng.shuffle(lens)
    return [[int(v) for v in rng.integers(0, 10**6, n)] for n in lens]


def test_partition_cache_near_shape_reuse(env):
    """a batch whose mean list length sits one 2^(1/4) step from a
    cached shape reuses that partition (no upload); a farther one uploads.
    Tiled kernel (the only one with a per-warp partition)."""
    rap, synth, oracle, torch = env
    B = 1000
    s = spec(0, 1, [node("sigridhash", [("s", 0)], salt=3, max_value=10**5)], [0])
    plan = rap.Plan(s, device=0)
    plan.set_kernel(rap.KERNEL_TILED)
    # 4*log2(mean): 6.16 -> 10.49 (key 10), 6.19 -> 10.52 (key 11), 9.0 -> 12.68 (key 13)
    ups = []
    for nnz in (6160, 6190, 6160, 9000):
        host = batch(B, sparse=[sparse_from_lists(_exact_nnz_lists(B, nnz, nnz))])
        raw = rap.DeviceBatch(host, "cuda:0")
        out = rap.DeviceOutput(plan, B, raw.sp_nnz, "cuda:0")
        plan.preprocess(raw, out)
        torch.cuda.synchronize()
        assert_parity(out.to_numpy(), oracle.run(s, host), f"nnz {nnz}")
        ups.append(plan.info()["partition_uploads"])
    plan.close()
    assert ups == [1, 1, 1, 2], ups


def test_graph_replay_after_partition_evictions(env, kmode):
    """a captured launch pins its partition slot, so eager calls
    over more than 8 other batch shapes (evicting every unpinned slot) do not
    change what the replay reads."""
    rap, synth, oracle, torch = env
    w = synth.c2_terabyte(0)
    plan = rap.Plan(w.spec, device=0)
    plan.set_kernel(kmode)
    host = synth.make_batch(w, 2500, seed=31)
    want = oracle.run(w.spec, host)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, 2500, raw.sp_nnz, "cuda:0")
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        plan.preprocess(raw, out, stream=st)
    st.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        plan.preprocess(raw, out, stream=st)
    others = []
    for i in range(10):  # 10 other shapes: every unpinned slot is evicted
        B = 1000 + 128 * i
        h = synth.make_batch(w, B, seed=40 + i)
        r = rap.DeviceBatch(h, "cuda:0")
        o = rap.DeviceOutput(plan, B, r.sp_nnz, "cuda:0")
        plan.preprocess(r, o)
        others.append((h, o))
    torch.cuda.synchronize()
    h, o = others[-1]
    assert_parity(o.to_numpy(), oracle.run(w.spec, h), "eager after evictions")
    out.values.fill_(-1)
    out.lengths.fill_(-1)
    g.replay()
    torch.cuda.synchronize()
    assert_parity(out.to_numpy(), want, "replay")
    plan.close()


@pytest.mark.parametrize("emitter", ["row", "col"])
def test_ngram_memo_providers_with_multi_id_rows(env, emitter, monkeypatch):
    """NGram outputs whose sources are memoised by single-id provider outputs
    (the generated kernel's register/shared memo path), over sources where
    some rows hold 2-3 ids: those rows leave the memo path for the generic
    NGram code (rb_fallback), in both generated emitters."""
    monkeypatch.setenv("RAP_JIT_EMIT", emitter)
    rng = np.random.default_rng(77)
    B = 1800
    sp = [sparse_from_lists(_lists(rng, B, 0, 10**6, max_len=1, p_null=0.1)) for _ in range(3)]
    # column 3: mostly single ids, a few rows with 2-3
    rows = _lists(rng, B, 0, 10**6, max_len=1, p_null=0.1)
    for i in range(0, B, 37):
        rows[i] = [int(v) for v in rng.integers(0, 10**6, 2 + i % 2)]
    sp.append(sparse_from_lists(rows))
    nodes = [node("sigridhash", [("s", i)], salt=20 + i, max_value=10**6 + i) for i in range(4)]
    nodes.append(node("ngram", [("s", 0), ("s", 1), ("s", 2)], n=3, salt=4, max_value=10**7))
    nodes.append(node("ngram", [("s", 1), ("s", 3), ("s", 2)], n=2, salt=5, max_value=2**40))
    nodes.append(node("ngram", [("s", 3), ("s", 0)], n=1, salt=6, max_value=999))
    s = spec(0, 4, nodes, list(range(7)))
    run_check(env, 3, s, batch(B, sparse=sp), ctx=emitter)
