"""Seeded synthetic Criteo-shaped workloads: graph specs + raw batches.

This module is the ONE piece shared by the oracle tests and the CUDA path
(DESIGN.md §5): it holds input descriptions and a counter-based random
generator, and none of the method's arithmetic.  Its mixer is the MurmurHash3
64-bit finaliser, deliberately not the SplitMix64 function the method uses
as its hash (reading R1).

Shapes follow PAPER.md: 13 dense + 26 sparse Criteo features (L1656-1657),
Table 2 total hash sizes 33.7M (Kaggle) / 177.9M (Terabyte) (L1610-1614),
Table 3 plan sizes (L1616-1621).  The recipe is in DESIGN.md §6.

Graph-spec format (plain dict):
  {"n_dense": D, "n_sparse": S,
   "nodes": [{"op": "fillnull"|"logit"|..., "inputs": [["d", c] | ["s", c] | ["n", i], ...],
              <op params: f_fill, i_fill, eps, lambda, borders, k, max_value, salt,
               x, lo, hi, n, keys, vals, map_default>}, ...],
   "outputs": [node index, ...]}
Raw batch (host numpy): {"n_rows", "dense": [f32[B]], "dense_valid": [u32[ceil(B/32)] | None],
  "sp_off": [i32[B+1]], "sp_val": [i64[...]], "sp_valid": [u32[...] | None]}.
"""
from __future__ import annotations

import math

import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
KAGGLE_TOTAL = 33_700_000
TB_TOTAL = 177_900_000


# ----------------------------------------------------------------------------- generator
def _fmix64(h):
    """MurmurHash3 fmix64 on a uint64 array (wrapping arithmetic)."""
    h = h.astype(np.uint64, copy=True)
    with np.errstate(over="ignore"):
        h ^= h >> np.uint64(33)
        h *= np.uint64(0xFF51AFD7ED558CCD)
        h ^= h >> np.uint64(33)
        h *= np.uint64(0xC4CEB9FE1A85EC53)
        h ^= h >> np.uint64(33)
    return h


def _stream_key(seed: int, *stream) -> np.uint64:
    k = np.array([seed & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64)
    for s in stream:
        if isinstance(s, str):
            s = sum((ord(ch) + 1) * 131 ** i for i, ch in enumerate(s)) & 0xFFFFFFFFFFFFFFFF
        with np.errstate(over="ignore"):
            k = _fmix64(k ^ _fmix64(np.array([s & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64) + np.uint64(0x5851F42D4C957F2D)))
    return k[0]


def bits(seed: int, stream, n: int, start: int = 0) -> np.ndarray:
    """n uint64 draws for (seed, stream, index=start..start+n-1)."""
    key = _stream_key(seed, *stream)
    idx = np.arange(start, start + n, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return _fmix64(_fmix64(idx * np.uint64(0xD6E8FEB86659FD93) + key) ^ key)


def uniform(seed: int, stream, n: int, start: int = 0) -> np.ndarray:
    """Uniform float64 in [0, 1) with 53 random bits."""
    return (bits(seed, stream, n, start) >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def normal(seed: int, stream, n: int, start: int = 0) -> np.ndarray:
    u1 = uniform(seed, tuple(stream) + ("bm1",), n, start)
    u2 = uniform(seed, tuple(stream) + ("bm2",), n, start)
    return np.sqrt(-2.0 * np.log1p(-u1)) * np.cos(2.0 * math.pi * u2)


def pack_bitmap(valid: np.ndarray) -> np.ndarray:
    """Arrow LSB validity bitmap as little-endian uint32 words."""
    b = np.packbits(valid.astype(np.uint8), bitorder="little")
    pad = (-len(b)) % 4
    if pad or len(b) == 0:
        b = np.concatenate([b, np.zeros(pad if len(b) else 4, dtype=np.uint8)])
    return b.view("<u4").astype(np.uint32)


def unpack_bitmap(words, n: int) -> np.ndarray:
    if words is None:
        return np.ones(n, dtype=bool)
    b = np.asarray(words, dtype="<u4").view(np.uint8)
    return np.unpackbits(b, bitorder="little")[:n].astype(bool)


# ----------------------------------------------------------------------------- feature shapes
def cardinalities(seed: int, n: int, total: int) -> np.ndarray:
    """Per-feature cardinality, log-uniform in [3, 4e7], rescaled so the table
    sizes sum to `total` (Table 2 total hash size, L1613-1614)."""
    u = uniform(seed, ("card",), n)
    c = np.exp(math.log(3.0) + u * (math.log(4e7) - math.log(3.0)))
    m = np.maximum(1, np.round(c * total / c.sum())).astype(np.int64)
    return m


def salts(seed: int, n: int, tag: str = "salt") -> list:
    return [int(x) for x in bits(seed, (tag,), n)]


def raw_id(rank: np.ndarray, feature: int) -> np.ndarray:
    """Fixed 32-bit bijection of Zipf ranks to raw ids (odd multiplier mod 2^32)."""
    r = rank.astype(np.uint64)
    with np.errstate(over="ignore"):
        v = (r * np.uint64(0x2C1B3C6D) + np.uint64((feature * 0x297A2D39) & 0xFFFFFFFF)) & np.uint64(0xFFFFFFFF)
    return v.astype(np.int64)


def zipf_ranks(seed: int, stream, n: int, card: int, s: float = 1.1) -> np.ndarray:
    """Zipf(s)-like ranks in [1, card] via the continuous power-law inverse CDF."""
    u = uniform(seed, stream, n)
    a = 1.0 - s
    top = card ** a
    r = np.floor((1.0 - u * (1.0 - top)) ** (1.0 / a))
    return np.clip(r, 1, card).astype(np.int64)


def poisson(seed: int, stream, n: int, mu: float) -> np.ndarray:
    """Poisson(mu) by inverse CDF over a float64 table."""
    kmax = int(mu + 12 * math.sqrt(mu) + 16)
    k = np.arange(kmax + 1)
    logp = -mu + k * math.log(mu) - np.array([math.lgamma(i + 1) for i in k])
    cdf = np.cumsum(np.exp(logp))
    cdf[-1] = 1.0
    u = uniform(seed, stream, n)
    return np.minimum(np.searchsorted(cdf, u, side="right"), kmax).astype(np.int64)


# ----------------------------------------------------------------------------- workloads
class Workload:
    """A graph spec plus what the raw-batch generator needs to know."""

    def __init__(self, name, spec, dense_kinds, sparse_card, sparse_mean=None, null_rate=0.2, multi_null=None):
        self.name = name
        self.spec = spec
        self.dense_kinds = dense_kinds          # per dense col: "unit" | "count"
        self.sparse_card = sparse_card          # per sparse col: cardinality for raw ids
        self.sparse_mean = sparse_mean          # None = single-valued; else per-col Poisson mean
        self.null_rate = null_rate              # per-col null prob ~ U[0, null_rate]
        self.multi_null = multi_null            # fixed null prob for multi-hot cols


def _n(op, inputs, **kw):
    d = {"op": op, "inputs": [list(x) for x in inputs]}
    d.update(kw)
    return d


def c1_kaggle(seed: int = 0) -> Workload:
    """Config 1: Criteo-Kaggle-shaped, 13 dense FillNull->Logit, 26 sparse
    SigridHash->Bucketize->FirstX (Table 3 Plan 0: 13x2 + 26x3 = 104 ops, L1618)."""
    nodes, outs = [], []
    for c in range(13):
        nodes.append(_n("fillnull", [("d", c)], f_fill=0.0))
        nodes.append(_n("logit", [("n", len(nodes) - 1)], eps=1e-6))
        outs.append(len(nodes) - 1)
    M = cardinalities(seed, 26, KAGGLE_TOTAL)
    sl = salts(seed, 26)
    for s in range(26):
        nodes.append(_n("sigridhash", [("s", s)], salt=sl[s], max_value=int(M[s])))
        borders = np.unique(np.floor(np.logspace(0, math.log10(max(int(M[s]), 2)), 1024))).astype(np.int64)
        borders = np.sort(np.concatenate([borders, np.full(1024 - len(borders), borders[-1])]))
        nodes.append(_n("bucketize", [("n", len(nodes) - 1)], borders=borders))
        nodes.append(_n("firstx", [("n", len(nodes) - 1)], x=1))
        outs.append(len(nodes) - 1)
    spec = {"n_dense": 13, "n_sparse": 26, "nodes": nodes, "outputs": outs}
    return Workload("criteo_kaggle_c1", spec, ["unit"] * 13, M.copy())


DENSE_BORDERS = np.array([0.5, 1.5, 2.5, 4.5, 8.5, 16.5, 32.5, 64.5, 128.5, 256.5, 512.5,
                          1024.5, 2048.5, 4096.5, 8192.5], dtype=np.float32)


def c2_terabyte(seed: int = 0, mapid_size: int = 4096, n_ngram: int = 8) -> Workload:
    """Config 2: Criteo-Terabyte-shaped full op graph:
    dense: FillNull(0) x13; Logit cols 0-5; BoxCox(lambda cycling) cols 6-12;
    cols 11-12 also Bucketize(15 borders)->OneHot(16).
    sparse x26: FillNull(0)->Clamp(0,2^32-1)->[MapId on 6]->SigridHash->[Bucketize on 4]->FirstX(1).
    NGram: 8 trigram features over 3 post-SigridHash sources each, M=10M.
    152 ops; 45 dense output columns; 34 sparse output features.
    n_ngram != 8: that many trigram features (sources cycling over the 26
    hashed features; the growing-NGram sweep, Fig 11)."""
    nodes, outs_dense, outs_sparse = [], [], []
    lambdas = [0.0, 0.25, 0.5, -0.5]
    fill_node = {}
    for c in range(13):
        nodes.append(_n("fillnull", [("d", c)], f_fill=0.0))
        fill_node[c] = len(nodes) - 1
        if c < 6:
            nodes.append(_n("logit", [("n", fill_node[c])], eps=1e-6))
        else:
            nodes.append(_n("boxcox", [("n", fill_node[c])], **{"lambda": lambdas[(c - 6) % 4]}))
        outs_dense.append(len(nodes) - 1)
    onehots = []
    for c in (11, 12):
        nodes.append(_n("bucketize", [("n", fill_node[c])], borders=DENSE_BORDERS.copy()))
        nodes.append(_n("onehot", [("n", len(nodes) - 1)], k=16))
        onehots.append(len(nodes) - 1)
    M = cardinalities(seed, 26, TB_TOTAL)
    sl = salts(seed, 26)
    mapid_feats = {1, 5, 9, 13, 17, 21}
    bucket_feats = {3, 11, 19, 24}
    hashed = {}
    for s in range(26):
        nodes.append(_n("fillnull", [("s", s)], i_fill=0))
        nodes.append(_n("clamp", [("n", len(nodes) - 1)], lo=0, hi=2**32 - 1))
        if s in mapid_feats:
            # keys = raw ids of the most frequent Zipf ranks (high hit rate), vals 1..size
            keys = raw_id(np.arange(1, mapid_size + 1), s)
            vals = np.arange(1, mapid_size + 1, dtype=np.int64)
            nodes.append(_n("mapid", [("n", len(nodes) - 1)], keys=keys, vals=vals, map_default=0))
        nodes.append(_n("sigridhash", [("n", len(nodes) - 1)], salt=sl[s], max_value=int(M[s])))
        hashed[s] = len(nodes) - 1
        if s in bucket_feats:
            borders = np.unique(np.floor(np.logspace(0, math.log10(max(int(M[s]), 2)), 1024))).astype(np.int64)
            borders = np.sort(np.concatenate([borders, np.full(1024 - len(borders), borders[-1])]))
            nodes.append(_n("bucketize", [("n", len(nodes) - 1)], borders=borders))
        nodes.append(_n("firstx", [("n", len(nodes) - 1)], x=1))
        outs_sparse.append(len(nodes) - 1)
    ng_salts = salts(seed, n_ngram, "ngram_salt")
    for g in range(n_ngram):
        srcs = [(3 * g) % 26, (3 * g + 1) % 26, (3 * g + 2) % 26]
        nodes.append(_n("ngram", [("n", hashed[s]) for s in srcs], n=3, salt=ng_salts[g], max_value=10_000_000))
        outs_sparse.append(len(nodes) - 1)
    spec = {"n_dense": 13, "n_sparse": 26, "nodes": nodes, "outputs": outs_dense + onehots + outs_sparse}
    kinds = ["unit"] * 6 + ["count"] * 7
    name = "criteo_terabyte_c2" if n_ngram == 8 else f"criteo_terabyte_c2_ngram{n_ngram}"
    return Workload(name, spec, kinds, M.copy())


def c4_multihot(seed: int = 0, n_features: int = 512, mean_len: float = 20.0, firstx: int = 32) -> Workload:
    """Config 4: 512 multi-hot sparse features, L ~ Poisson(mu_f), mu_f = mean_len*w_f,
    w_f ~ LogNormal(0, 0.5) normalised to mean 1; FillNull(0)->Clamp->SigridHash->FirstX(32)."""
    w = np.exp(0.5 * normal(seed, ("mu",), n_features))
    w = w / w.mean()
    mu = mean_len * w
    M = cardinalities(seed, n_features, TB_TOTAL)
    sl = salts(seed, n_features)
    nodes, outs = [], []
    for s in range(n_features):
        nodes.append(_n("fillnull", [("s", s)], i_fill=0))
        nodes.append(_n("clamp", [("n", len(nodes) - 1)], lo=0, hi=2**32 - 1))
        nodes.append(_n("sigridhash", [("n", len(nodes) - 1)], salt=sl[s], max_value=int(M[s])))
        nodes.append(_n("firstx", [("n", len(nodes) - 1)], x=firstx))
        outs.append(len(nodes) - 1)
    spec = {"n_dense": 0, "n_sparse": n_features, "nodes": nodes, "outputs": outs}
    return Workload("multihot_c4", spec, [], M.copy(), sparse_mean=mu, multi_null=0.05)


# Table 3 (L1616-1621): (dense, sparse) input features and total ops.  Plan 3's
# "9.80 ops/feature" and "1548 ops" disagree (156 x 9.80 = 1528.8, reading
# R18); the generator builds 1548.
PLAN_SHAPES = {2: (26, 52, 384), 3: (52, 104, 1548)}


def plan_graph(plan: int, seed: int = 0) -> Workload:
    """Table 3 Plan 2 / Plan 3-shaped op graph (NEXT-4): the config-2 recipe
    scaled to the plan's features, extended until it has exactly the plan's
    op count.  Base chains: dense FillNull -> Logit | BoxCox; sparse FillNull
    -> Clamp -> SigridHash -> FirstX(1).  Extras, added round robin: MapId
    before a SigridHash, Bucketize after it, an NGram over three hashed
    sources, a dense Bucketize -> OneHot(16), and a re-hash (Clamp ->
    SigridHash) deepening a sparse chain (not the canonical stage order: the
    kernels' generic paths)."""
    n_dense, n_sparse, n_ops = PLAN_SHAPES[plan]
    lambdas = [0.0, 0.25, 0.5, -0.5]
    mapid = [False] * n_sparse
    bucket = [False] * n_sparse
    rehash = [0] * n_sparse
    onehot = [0] * n_dense
    ngrams = []
    remaining = n_ops - (2 * n_dense + 4 * n_sparse)
    i = 0
    while remaining > 0:
        kind = i % 5
        s, d = (i * 7) % n_sparse, (i * 3) % n_dense
        if kind == 0 and not mapid[s]:
            mapid[s] = True
            remaining -= 1
        elif kind == 1 and not bucket[s]:
            bucket[s] = True
            remaining -= 1
        elif kind == 2:
            ngrams.append([s, (s + 1) % n_sparse, (s + 5) % n_sparse])
            remaining -= 1
        elif kind == 3 and remaining >= 2 and onehot[d] < 1 and d % 4 == 3:
            onehot[d] += 1
            remaining -= 2
        elif kind == 4 and remaining >= 2 and rehash[s] < 6:
            rehash[s] += 1
            remaining -= 2
        i += 1
    nodes, outs_dense, outs_vec, outs_sparse = [], [], [], []
    for c in range(n_dense):
        nodes.append(_n("fillnull", [("d", c)], f_fill=0.0))
        f = len(nodes) - 1
        if c % 2 == 0:
            nodes.append(_n("logit", [("n", f)], eps=1e-6))
        else:
            nodes.append(_n("boxcox", [("n", f)], **{"lambda": lambdas[(c // 2) % 4]}))
        outs_dense.append(len(nodes) - 1)
        for k in range(onehot[c]):
            nodes.append(_n("bucketize", [("n", f)], borders=(DENSE_BORDERS * (1 + k)).astype(np.float32)))
            nodes.append(_n("onehot", [("n", len(nodes) - 1)], k=16))
            outs_vec.append(len(nodes) - 1)
    M = cardinalities(seed, n_sparse, TB_TOTAL)
    sl = salts(seed, n_sparse, f"plan{plan}_salt")
    hashed = {}
    for s in range(n_sparse):
        nodes.append(_n("fillnull", [("s", s)], i_fill=0))
        nodes.append(_n("clamp", [("n", len(nodes) - 1)], lo=0, hi=2**32 - 1))
        if mapid[s]:
            keys = raw_id(np.arange(1, 1025), s)
            nodes.append(_n("mapid", [("n", len(nodes) - 1)], keys=keys, vals=np.arange(1, 1025, dtype=np.int64),
                            map_default=0))
        nodes.append(_n("sigridhash", [("n", len(nodes) - 1)], salt=sl[s], max_value=int(M[s])))
        hashed[s] = len(nodes) - 1
        for r in range(rehash[s]):
            nodes.append(_n("clamp", [("n", len(nodes) - 1)], lo=0, hi=max(int(M[s]) - 1 - r, 0)))
            nodes.append(_n("sigridhash", [("n", len(nodes) - 1)], salt=sl[s] ^ (r + 1), max_value=int(M[s])))
        if bucket[s]:
            borders = np.unique(np.floor(np.logspace(0, math.log10(max(int(M[s]), 2)), 256))).astype(np.int64)
            nodes.append(_n("bucketize", [("n", len(nodes) - 1)], borders=borders))
        nodes.append(_n("firstx", [("n", len(nodes) - 1)], x=1))
        outs_sparse.append(len(nodes) - 1)
    ng_salts = salts(seed, max(len(ngrams), 1), f"plan{plan}_ngram")
    for g, srcs in enumerate(ngrams):
        nodes.append(_n("ngram", [("n", hashed[x]) for x in srcs], n=3, salt=ng_salts[g], max_value=10_000_000))
        outs_sparse.append(len(nodes) - 1)
    assert len(nodes) == n_ops, (len(nodes), n_ops)
    spec = {"n_dense": n_dense, "n_sparse": n_sparse, "nodes": nodes,
            "outputs": outs_dense + outs_vec + outs_sparse}
    kinds = ["unit" if c % 2 == 0 else "count" for c in range(n_dense)]
    return Workload(f"table3_plan{plan}", spec, kinds, M.copy())


def plan2(seed: int = 0) -> Workload:
    return plan_graph(2, seed)


def plan3(seed: int = 0) -> Workload:
    return plan_graph(3, seed)


WORKLOADS = {"c1": c1_kaggle, "c2": c2_terabyte, "c4": c4_multihot, "plan2": plan2, "plan3": plan3}


# ----------------------------------------------------------------------------- raw batches
def dense_column(seed: int, c: int, kind: str, n: int, null_rate: float = 0.2, row0: int = 0):
    """One dense column: values f32[n], validity u32 bitmap.  Nulls are encoded
    50/50 as a cleared validity bit (slot holds junk) or as a NaN payload."""
    p = null_rate * uniform(seed, ("dense_p", c), 1)[0]
    null = uniform(seed, ("dense_null", c), n, row0) < p
    as_nan = uniform(seed, ("dense_enc", c), n, row0) < 0.5
    if kind == "unit":
        # Beta(2,5) = 2nd order statistic of 6 uniforms; plus 1% exact 0 and 1% exact 1
        u = np.stack([uniform(seed, ("dense_u", c, i), n, row0) for i in range(6)])
        x = np.sort(u, axis=0)[1]
        e = uniform(seed, ("dense_edge", c), n, row0)
        x = np.where(e < 0.01, 0.0, np.where(e > 0.99, 1.0, x))
    else:
        z = normal(seed, ("dense_z", c), n, row0)
        x = np.floor(np.exp(1.5 + 1.5 * z))
    x = x.astype(np.float32)
    valid = ~(null & ~as_nan)
    x = np.where(null & as_nan, np.float32(np.nan), x)
    x = np.where(~valid, np.float32(12345.0), x).astype(np.float32)   # junk in null slots
    return x, pack_bitmap(valid)


def sparse_column(seed: int, s: int, card: int, n: int, mean=None, null_p=None, null_rate: float = 0.2,
                  null_segments: bool = False, base_offset: int = 0, row0: int = 0):
    """One Arrow list<int64> column: offsets i32[n+1], values i64, validity u32 bitmap."""
    p = null_p if null_p is not None else null_rate * uniform(seed, ("sp_p", s), 1)[0]
    null = uniform(seed, ("sp_null", s), n, row0) < p
    if mean is None:
        lens = np.ones(n, dtype=np.int64)
    else:
        lens = poisson(seed, ("sp_len", s, row0), n, float(mean))
    if not null_segments:
        lens = np.where(null, 0, lens)
    total = int(lens.sum())
    ids = raw_id(zipf_ranks(seed, ("sp_id", s, row0), total, int(card)), s)
    off = np.empty(n + 1, dtype=np.int64)
    off[0] = base_offset
    np.cumsum(lens, out=off[1:])
    off[1:] += base_offset
    vals = np.concatenate([np.full(base_offset, -7, dtype=np.int64), ids]) if base_offset else ids
    return off.astype(np.int32), vals.astype(np.int64), pack_bitmap(~null)


def make_batch(w: Workload, n_rows: int, seed: int = 1, null_segments: bool = False, base_offset: int = 0,
               drop_bitmaps: bool = False):
    """Raw columnar batch for workload w (host numpy arrays)."""
    spec = w.spec
    dense, dvalid = [], []
    for c in range(spec["n_dense"]):
        x, v = dense_column(seed, c, w.dense_kinds[c], n_rows, w.null_rate)
        dense.append(x)
        dvalid.append(None if drop_bitmaps else v)
    soff, sval, svalid = [], [], []
    for s in range(spec["n_sparse"]):
        mean = None if w.sparse_mean is None else w.sparse_mean[s]
        o, v, b = sparse_column(seed, s, w.sparse_card[s], n_rows, mean, w.multi_null, w.null_rate,
                                null_segments, base_offset)
        soff.append(o)
        sval.append(v)
        svalid.append(None if drop_bitmaps else b)
    return {"n_rows": n_rows, "dense": dense, "dense_valid": dvalid, "sp_off": soff, "sp_val": sval,
            "sp_valid": svalid}


def output_dims(spec) -> tuple:
    """(dense output columns, sparse output features) implied by a spec, by the
    type rules of DESIGN.md §3 (no arithmetic)."""
    d = f = 0
    for o, t in zip(spec["outputs"], output_types(spec)):
        if t == "D":
            d += 1
        elif t == "V":
            d += spec["nodes"][o]["k"]
        else:
            f += 1
    return d, f


def output_types(spec) -> list:
    """Type of every output node: 'D' dense scalar, 'V' OneHot vector, 'I' id
    list (a sparse output), by the type rules of DESIGN.md §3."""
    types = {}

    def tin(kind, idx):
        return {"d": "D", "s": "I"}[kind] if kind != "n" else types[idx]

    def typ(i):
        if i in types:
            return types[i]
        nd = spec["nodes"][i]
        for k, idx in nd["inputs"]:
            if k == "n":
                typ(idx)
        op = nd["op"]
        t0 = tin(*nd["inputs"][0])
        t = {"fillnull": t0, "logit": "D", "boxcox": "D", "onehot": "V", "bucketize": "I"}.get(op, "I")
        types[i] = t
        return t

    return [typ(o) for o in spec["outputs"]]


def algorithmic_bytes(spec, batch, n_values_out: int) -> int:
    """Bytes the method must move for one batch: every raw byte read once, every
    output byte written once.  Params/tables count as 0."""
    B = int(batch["n_rows"])
    used_d, used_s = set(), set()
    for nd in spec["nodes"]:
        for k, idx in nd["inputs"]:
            if k == "d":
                used_d.add(idx)
            elif k == "s":
                used_s.add(idx)
    rd = 0
    for c in used_d:
        rd += 4 * B + (0 if batch["dense_valid"][c] is None else (B + 7) // 8)
    for s in used_s:
        off = batch["sp_off"][s]
        rd += 4 * (B + 1) + 8 * int(off[-1] - off[0]) + (0 if batch["sp_valid"][s] is None else (B + 7) // 8)
    D, F = output_dims(spec)
    wr = 4 * B * D + 4 * B * F + 8 * (B * F + 1) + 8 * int(n_values_out)
    return int(rd + wr)
