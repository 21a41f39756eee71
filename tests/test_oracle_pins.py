"""Pins for the CPU oracle (runs with -m "not gpu").

Every test ties the oracle to something other than itself: published vectors,
library routines (numpy / torch / scipy), closed forms, invariants, hand-worked
examples or brute force.  Citations: PAPER.md Table 1 L440-463 for the ops,
DESIGN.md §3 for the readings R1-R17.
"""
import itertools
import json
import math
import os

import numpy as np
import pytest

from tests.helpers import batch, dense_from_values, node, sparse_from_lists, spec, split_jagged

GOLD = os.path.join(os.path.dirname(__file__), "golden")
GAMMA = 0x9E3779B97F4A7C15
M64 = 2**64 - 1


def _load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def s64(u):
    """uint64 -> int64 (two's complement)."""
    u &= M64
    return u - 2**64 if u >= 2**63 else u


def f32(x):
    return float(np.float32(x))


def ulp_diff(a, b):
    a = np.array([a], dtype=np.float32).view(np.int32)[0].astype(np.int64)
    b = np.array([b], dtype=np.float32).view(np.int32)[0].astype(np.int64)
    if a < 0:
        a = -(2**31) - a
    if b < 0:
        b = -(2**31) - b
    return abs(int(a) - int(b))


# ------------------------------------------------------------------ H and reduce (R1, R2)
def test_H_published_splitmix64_vectors(orc):
    g = _load("splitmix64_vectors.json")
    assert orc.H(0) == int(g["seed_0_first"], 16)
    seq = [int(v) for v in g["seed_1234567_first_three"]]
    # SplitMix64 output k (k = 0, 1, 2) of seed s is H(s + k * gamma)
    for k, want in enumerate(seq):
        assert orc.H((1234567 + k * GAMMA) & M64) == want


def test_reduce_closed_forms(orc):
    rng = np.random.default_rng(0)
    for h in [0, 1, 2**63, M64] + [int(v) for v in rng.integers(0, 2**63, 50, dtype=np.int64)]:
        assert orc.reduce(h, 1) == 0
        assert orc.reduce(h, 2**62) == h >> 2
        assert orc.reduce(h, 2**32) == h >> 32
        for M in (3, 1000, 10_131_227, 2**63 - 1):
            r = orc.reduce(h, M)
            assert 0 <= r < M
            assert r == (h * M) >> 64          # big-int brute force


def test_sigridhash_composition_pinned_to_splitmix64(orc):
    """With M = 2^62 the reduction is h >> 2, and x / salt are chosen so that
    every H argument is a seed whose SplitMix64 output is published."""
    g = _load("splitmix64_vectors.json")
    h0 = int(g["seed_0_first"], 16)
    seq = [int(v) for v in g["seed_1234567_first_three"]]
    # salt 0: H(H(0) ^ x) with x = H(0) ^ 1234567  ->  H(1234567)
    assert orc.sigridhash(s64(h0 ^ 1234567), 0, 2**62) == seq[0] >> 2
    # salt 1234567: H(H(1234567) ^ x) with x = H(1234567) ^ (1234567 + gamma)
    assert orc.sigridhash(s64(seq[0] ^ ((1234567 + GAMMA) & M64)), 1234567, 2**62) == seq[1] >> 2


def test_sigridhash_spec_goldens(orc):
    for c in _load("spec_goldens.json")["sigridhash"]:
        assert orc.sigridhash(c["x"], c["salt"], c["M"]) == c["y"]


def test_sigridhash_range_and_m1(orc):
    rng = np.random.default_rng(1)
    for x in rng.integers(-2**63, 2**63 - 1, 200, dtype=np.int64):
        assert orc.sigridhash(int(x), 77, 1) == 0
        assert 0 <= orc.sigridhash(int(x), 77, 12345) < 12345


# ------------------------------------------------------------------ NGram (R7)
def test_ngram_chaining_pinned_to_splitmix64(orc):
    g = _load("splitmix64_vectors.json")
    h0 = int(g["seed_0_first"], 16)
    seq = [int(v) for v in g["seed_1234567_first_three"]]
    a = s64(h0 ^ 1234567)                                  # H(H(0)^a) = seq[0]
    b = s64(seq[0] ^ ((1234567 + GAMMA) & M64))            # H(seq[0]^b) = seq[1]
    c = s64(seq[1] ^ ((1234567 + 2 * GAMMA) & M64))        # H(seq[1]^c) = seq[2]
    assert orc.ngram([a], 1, 0, 2**62) == [seq[0] >> 2]
    assert orc.ngram([a, b], 2, 0, 2**62) == [seq[1] >> 2]
    assert orc.ngram([a, b, c], 3, 0, 2**62) == [seq[2] >> 2]


def test_ngram_spec_goldens(orc):
    for c in _load("spec_goldens.json")["ngram"]:
        assert orc.ngram(c["c"], c["n"], c["salt"], c["M"]) == c["out"]


def test_ngram_count_closed_form(orc):
    h = _load("hand_examples.json")["ngram_counts"]
    for L, want in zip(h["L"], h["count"]):
        assert len(orc.ngram(list(range(L)), h["n"], 9, 1000)) == want
    for n in range(1, 9):
        for L in range(0, 12):
            assert len(orc.ngram(list(range(100, 100 + L)), n, 3, 97)) == max(0, L - n + 1)


def test_ngram_n1_equals_sigridhash(orc):
    rng = np.random.default_rng(2)
    xs = [int(v) for v in rng.integers(-2**40, 2**40, 64)]
    for salt, M in [(5, 1000), (2**64 - 3, 10_000_000), (0, 1)]:
        assert orc.ngram(xs, 1, salt, M) == [orc.sigridhash(x, salt, M) for x in xs]


def test_ngram_window_locality(orc):
    """Window j depends only on c[j:j+n] (catches shifted / reversed indices)."""
    rng = np.random.default_rng(3)
    c = [int(v) for v in rng.integers(0, 2**40, 20)]
    for n in (2, 3, 5):
        full = orc.ngram(c, n, 11, 10**9)
        for j in range(len(c) - n + 1):
            assert full[j] == orc.ngram(c[j:j + n], n, 11, 10**9)[0]
        # order matters: reversing a window changes the hash (with overwhelming probability)
        assert orc.ngram(c[:n][::-1], n, 11, 10**9)[0] != full[0]


# ------------------------------------------------------------------ Bucketize (R4)
def test_bucketize_hand_example(orc):
    h = _load("hand_examples.json")["bucketize"]
    for x, y in zip(h["x"], h["y"]):
        assert orc.bucketize_f(float(x), h["borders"]) == y


def test_bucketize_matches_numpy_and_torch(orc):
    import torch

    rng = np.random.default_rng(4)
    borders = np.sort(rng.choice(np.arange(-20, 20, 0.5, dtype=np.float32), 17)).astype(np.float32)
    xs = np.concatenate([rng.uniform(-25, 25, 300).astype(np.float32), borders, [np.inf, -np.inf]]).astype(np.float32)
    want_np = np.searchsorted(borders, xs, side="right")
    want_t = torch.bucketize(torch.from_numpy(xs), torch.from_numpy(borders), right=True).numpy()
    got = [orc.bucketize_f(float(x), borders) for x in xs]
    assert list(want_np) == got
    assert list(want_t) == got
    ib = np.sort(rng.integers(-2**62, 2**62, 33, dtype=np.int64))
    ib[5] = ib[6]  # a duplicate border
    xi = np.concatenate([rng.integers(-2**63, 2**63 - 1, 300, dtype=np.int64), ib])
    assert list(np.searchsorted(ib, xi, side="right")) == [orc.bucketize_i(int(x), ib) for x in xi]


# ------------------------------------------------------------------ Logit (R11)
def test_logit_hand_values(orc):
    h = _load("hand_examples.json")["logit_eps_1e-6"]
    for x, y in zip(h["x"], h["y"]):
        got = orc.logit(float(x), 1e-6)
        if y == "nan":
            assert math.isnan(got)
        else:
            assert ulp_diff(got, f32(y)) <= 1, (x, got, y)
    assert orc.logit(0.5, 1e-6) == 0.0
    assert ulp_diff(orc.logit(0.75, 1e-6), f32(math.log(3.0))) <= 1


def test_logit_matches_torch(orc):
    import torch

    rng = np.random.default_rng(5)
    xs = np.concatenate([rng.uniform(-0.1, 1.1, 2000), rng.uniform(0, 1e-5, 100), 1 - rng.uniform(0, 1e-5, 100),
                         [0.0, 1.0, 0.5, np.nan, np.inf, -np.inf]]).astype(np.float32)
    for eps in (1e-6, 1e-3, 0.25):
        want = torch.logit(torch.from_numpy(xs), eps=eps).numpy()
        for x, w in zip(xs, want):
            g = orc.logit(float(x), eps)
            if math.isnan(w):
                assert math.isnan(g)
            else:
                assert ulp_diff(g, w) <= 2, (x, eps, g, w)


# ------------------------------------------------------------------ BoxCox (R12)
def test_boxcox_matches_scipy_fp64(orc):
    from scipy.special import boxcox

    rng = np.random.default_rng(6)
    xs = np.concatenate([np.floor(np.exp(1.5 + 1.5 * rng.standard_normal(500))), rng.uniform(0, 3, 500),
                         1 + rng.uniform(-1e-3, 1e-3, 100), [0.0, 1.0, 2.0, 1e-30, 1e30]]).astype(np.float32)
    for lam in (0.0, 0.25, 0.5, -0.5, 1.0, -1.0, 2.0):
        want = boxcox(xs.astype(np.float64), lam)
        for x, w in zip(xs, want):
            g = orc.boxcox(float(x), lam)
            w = float(np.float32(w)) if abs(w) > 3.4e38 else w   # beyond f32 range -> +-inf
            if math.isnan(w) or math.isinf(w):
                assert (math.isnan(g) and math.isnan(w)) or g == w, (x, lam, g, w)
            elif w == 0.0:
                assert g == 0.0
            else:
                assert abs(g - w) <= 1e-5 * abs(w), (x, lam, g, w)


def test_boxcox_closed_forms(orc):
    for c in _load("hand_examples.json")["boxcox"]["cases"]:
        x, lam, y = c
        g = orc.boxcox(x, lam)
        if y == "nan":
            assert math.isnan(g)
        elif y == "-inf":
            assert g == -math.inf
        else:
            assert abs(g - y) <= 1e-6 * max(1, abs(y)), c
    rng = np.random.default_rng(7)
    for x in rng.uniform(0.01, 100, 300).astype(np.float32):
        x = float(x)
        assert orc.boxcox(x, 0.0) == f32(math.log(x))
        assert abs(orc.boxcox(x, 1.0) - (x - 1)) <= 1e-5 * max(1e-3, abs(x - 1)) + 1e-7
        assert abs(orc.boxcox(x, 0.5) - 2 * (math.sqrt(x) - 1)) <= 1e-5 * max(1e-3, abs(2 * (math.sqrt(x) - 1))) + 1e-7
        assert abs(orc.boxcox(x, -1.0) - (1 - 1 / x)) <= 1e-5 * max(1e-3, abs(1 - 1 / x)) + 1e-7
    ys = [orc.boxcox(float(x), 0.25) for x in np.linspace(0.01, 50, 500, dtype=np.float32)]
    assert all(a <= b for a, b in zip(ys, ys[1:]))


# ------------------------------------------------------------------ graph-level (orc_run)
def test_hand_example_fillnull_firstx(orc):
    h = _load("hand_examples.json")["fillnull_firstx"]
    sp = sparse_from_lists(h["rows"])
    g = spec(0, 1, [node("fillnull", [("s", 0)], i_fill=h["fill"]), node("firstx", [("n", 0)], x=h["x"])], [1])
    r = orc.run(g, batch(4, sparse=[sp]))
    assert r["status"] == "OK"
    assert list(r["lengths"]) == h["lengths"]
    assert list(r["offsets"]) == h["offsets"]
    assert list(r["values"]) == h["values"]


def test_null_list_without_fill_is_empty_even_with_payload(orc):
    h = _load("hand_examples.json")["null_without_fill"]
    for payload in (None, [111, 222]):
        sp = sparse_from_lists(h["rows"], base_offset=3, null_payload=payload)
        g = spec(0, 1, [node("firstx", [("s", 0)], x=10)], [0])
        r = orc.run(g, batch(3, sparse=[sp]))
        assert list(r["lengths"]) == h["lengths"]
        assert list(r["values"]) == h["values"]


def _brute_chain(rows, fill, x):
    out = []
    for r in rows:
        if r is None:
            r = None if fill is None else [fill]
        out.append(None if r is None else r[:x])
    return out


def test_brute_force_tiny_lists(orc):
    """Every list of length <= 3 over a 3-symbol alphabet plus null, FillNull
    on/off, FirstX(x) for x in 0..4, NGram(n) for n in 1..4 over (chain, raw)."""
    alphabet = [0, 7, -3]
    lists = [None] + [list(p) for L in range(4) for p in itertools.product(alphabet, repeat=L)]
    rows = lists
    B = len(rows)
    sp = sparse_from_lists(rows, base_offset=1)
    sp2 = sparse_from_lists(rows[::-1])
    for use_fill in (False, True):
        for x in range(5):
            for n in range(1, 5):
                nodes = []
                src = ("s", 0)
                if use_fill:
                    nodes.append(node("fillnull", [src], i_fill=9))
                    src = ("n", len(nodes) - 1)
                nodes.append(node("firstx", [src], x=x))
                chain = len(nodes) - 1
                nodes.append(node("ngram", [("n", chain), ("s", 1)], n=n, salt=4, max_value=1000))
                g = spec(0, 2, nodes, [chain, len(nodes) - 1])
                r = orc.run(g, batch(B, sparse=[sp, sp2]))
                feats = split_jagged(r, B)
                want_chain = _brute_chain(rows, 9 if use_fill else None, x)
                assert feats[0] == [[] if v is None else v for v in want_chain]
                for b in range(B):
                    c = (want_chain[b] or []) + (rows[::-1][b] or [])
                    cnt = max(0, len(c) - n + 1)
                    want = [orc.ngram(c[j:j + n], n, 4, 1000)[0] for j in range(cnt)]
                    assert feats[1][b] == want
                # jagged invariants
                o = r["offsets"]
                assert o[0] == 0 and all(o[i] <= o[i + 1] for i in range(len(o) - 1))
                assert o[-1] == sum(r["lengths"]) == len(r["values"])


def test_clamp_mapid_onehot_against_library(orc):
    import torch

    rng = np.random.default_rng(8)
    rows = [list(rng.integers(-50, 50, rng.integers(0, 5))) if rng.random() > 0.2 else None for _ in range(300)]
    sp = sparse_from_lists(rows)
    keys = np.array(rng.choice(np.arange(-50, 50), 40, replace=False), dtype=np.int64)
    vals = rng.integers(1000, 2000, 40)
    g = spec(0, 1, [node("clamp", [("s", 0)], lo=-10, hi=20),
                    node("mapid", [("s", 0)], keys=keys, vals=vals, map_default=-1),
                    node("onehot", [("s", 0)], k=16)], [0, 1, 2])
    r = orc.run(g, batch(len(rows), sparse=[sp]))
    feats = split_jagged(r, len(rows))
    d = dict(zip(keys.tolist(), vals.tolist()))
    for b, row in enumerate(rows):
        row = row or []
        assert feats[0][b] == list(np.clip(np.array(row, dtype=np.int64), -10, 20))
        assert feats[1][b] == [d.get(int(v), -1) for v in row]
        inr = sorted({int(v) for v in row if 0 <= v < 16})
        want = np.zeros(16, dtype=np.float32)
        if inr:
            want = torch.nn.functional.one_hot(torch.tensor(inr), 16).sum(0).clamp(max=1).float().numpy()
        assert np.array_equal(r["dense"][b], want)
    # single-id case is exactly F.one_hot
    ids = rng.integers(0, 16, 50)
    sp1 = sparse_from_lists([[int(i)] for i in ids])
    r1 = orc.run(spec(0, 1, [node("onehot", [("s", 0)], k=16)], [0]), batch(50, sparse=[sp1]))
    assert np.array_equal(r1["dense"], torch.nn.functional.one_hot(torch.from_numpy(ids), 16).float().numpy())


def test_dense_chain_fillnull_and_dense_bucketize(orc):
    vals = [0.25, None, float("nan"), float("inf"), -float("inf"), 0.75, 3.0, None]
    d = dense_from_values(vals)
    g = spec(1, 0, [node("fillnull", [("d", 0)], f_fill=0.5),
                    node("logit", [("d", 0)], eps=1e-6),
                    node("bucketize", [("d", 0)], borders=np.array([0.0, 0.5, 1.0], dtype=np.float32)),
                    node("bucketize", [("n", 0)], borders=np.array([0.0, 0.5, 1.0], dtype=np.float32))],
             [0, 1, 2, 3])
    r = orc.run(g, batch(len(vals), dense=[d]))
    filled = r["dense"][:, 0]
    assert not np.isnan(filled).any()
    assert list(filled) == [0.25, 0.5, 0.5, np.inf, -np.inf, 0.75, 3.0, 0.5]
    raw_logit = r["dense"][:, 1]
    assert np.isnan(raw_logit[1]) and np.isnan(raw_logit[2]) and np.isnan(raw_logit[7])   # null -> NaN (R14)
    feats = split_jagged(r, len(vals))
    assert feats[0] == [[1], [0], [0], [3], [0], [2], [3], [0]]     # NaN -> bucket 0; each row length 1
    assert feats[1] == [[1], [2], [2], [3], [0], [2], [3], [2]]


def test_error_codes(orc):
    ok = spec(1, 1, [node("fillnull", [("d", 0)], f_fill=0.0)], [0])
    assert orc.validate(ok)[0] == "OK"
    cases = {
        "INVALID_GRAPH": [
            spec(1, 1, [node("logit", [("s", 0)], eps=1e-6)], [0]),                       # type mismatch
            spec(1, 1, [node("firstx", [("n", 1)], x=1), node("firstx", [("n", 0)], x=1)], [0]),   # cycle
            spec(1, 1, [node("firstx", [("s", 3)], x=1)], [0]),                            # bad raw ref
            spec(1, 1, [node("firstx", [("s", 0)], x=1)], [5]),                            # bad output
            spec(1, 1, [node(42, [("s", 0)])], [0]),                                       # unknown op
        ],
        "INVALID_PARAM": [
            spec(1, 0, [node("logit", [("d", 0)], eps=0.5)], [0]),
            spec(1, 0, [node("fillnull", [("d", 0)], f_fill=float("nan"))], [0]),
            spec(1, 0, [node("boxcox", [("d", 0)], **{"lambda": float("inf")})], [0]),
            spec(1, 0, [node("bucketize", [("d", 0)], borders=np.array([1.0, 0.0], dtype=np.float32))], [0]),
            spec(0, 1, [node("sigridhash", [("s", 0)], salt=1, max_value=0)], [0]),
            spec(0, 1, [node("firstx", [("s", 0)], x=-1)], [0]),
            spec(0, 1, [node("clamp", [("s", 0)], lo=5, hi=4)], [0]),
            spec(0, 1, [node("ngram", [("s", 0)], n=9, salt=1, max_value=10)], [0]),
            spec(0, 1, [node("mapid", [("s", 0)], keys=[1, 1], vals=[2, 3])], [0]),
            spec(0, 1, [node("onehot", [("s", 0)], k=0)], [0]),
        ],
    }
    for want, specs in cases.items():
        for s in specs:
            assert orc.validate(s)[0] == want, s


def test_c2_workload_invariants(orc):
    from paper_conf_asplos_wangwdz0d24_b200 import synth

    w = synth.c2_terabyte(0)
    st, D, F = orc.validate(w.spec)
    assert (st, D, F) == ("OK", 45, 34)
    assert synth.output_dims(w.spec) == (45, 34)
    assert len(w.spec["nodes"]) == 152           # SURVEY §8(d) op count
    B = 3000
    b = synth.make_batch(w, B, seed=3)
    r = orc.run(w.spec, b)
    L, O = r["lengths"], r["offsets"]
    assert O[0] == 0 and np.all(np.diff(O) >= 0) and O[-1] == L.sum() == len(r["values"])
    # FillNull makes every single-valued sparse feature exactly one id per row;
    # each trigram over three single-valued sources has exactly one window.
    assert np.all(L == 1)
    assert not np.isnan(r["dense"][:, :6]).any()
    onehot = r["dense"][:, 13:]
    assert np.all(onehot.reshape(B, 2, 16).sum(-1) == 1)


def test_spec_goldens_regenerate():
    """spec_goldens.json is what the committed big-int generator writes, and the
    generator's H is itself pinned to the published SplitMix64 vectors."""
    import importlib.util
    import os

    p = os.path.join(os.path.dirname(__file__), "golden", "make_spec_goldens.py")
    sp = importlib.util.spec_from_file_location("make_spec_goldens", p)
    m = importlib.util.module_from_spec(sp)
    sp.loader.exec_module(m)
    g = _load("splitmix64_vectors.json")
    assert m.H(0) == int(g["seed_0_first"], 16)
    have = _load("spec_goldens.json")
    want = m.goldens()
    assert have["sigridhash"] == want["sigridhash"] and have["ngram"] == want["ngram"]


def test_cast_int32_reading_r13():
    """Cast (Table 1, reading R13): an id cast to int32 keeps its low 32
    bits as a two's-complement value -- numpy's astype, checked on hand-worked
    values (the GPU int32 emission is compared with the oracle's ids cast this way)."""
    ids = np.array([5, -1, 2**31 - 1, 2**31, 2**31 + 5, 2**32 + 7, -(2**31) - 1, -(2**63)], dtype=np.int64)
    want = [5, -1, 2147483647, -2147483648, -2147483643, 7, 2147483647, 0]
    assert ids.astype(np.int32).tolist() == want
