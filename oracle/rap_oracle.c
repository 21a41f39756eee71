/*
 * rap_oracle.c — plain, slow, row-by-row CPU oracle.  TEST INFRASTRUCTURE ONLY
 * (see rap_oracle.h for who may load it).  Builds with:
 *   gcc -std=c11 -O1 -ffp-contract=off -fno-fast-math -fPIC -shared -lm
 *
 * Every operator follows the one-line definition of PAPER.md Table 1
 * (L440-463) plus the reading listed in DESIGN.md §3 (the paper defines no
 * operator beyond that line).  No blocking, no fusion, no reordering: for each
 * row, each node of the DAG (§2.3) is evaluated once, in
 * topological order, from its inputs' per-row values.
 *
 * Pins (tests/test_oracle_pins.py) — what fixes each function independently
 * of this file:
 *   orc_H           published SplitMix64 output vectors (seed 0, seed 1234567)
 *   orc_reduce      M=1 -> 0, M=2^62 -> h>>2, big-int brute force
 *   orc_sigridhash  composition pinned to the SplitMix64 vectors via M=2^62
 *   orc_logit       torch.logit(x, eps) on f32; logit(0.5)=0; logit(.75)=ln 3
 *   orc_boxcox      scipy.special.boxcox (fp64); lambda 0/1/0.5/-1 closed forms
 *   orc_bucketize_* numpy.searchsorted(side='right'); hand example
 *   FirstX/Clamp    closed forms, prefix property
 *   orc_ngram       count = max(0, L-n+1); n=1 == SigridHash; brute force
 *   MapId           Python dict brute force
 *   OneHot          torch.nn.functional.one_hot for single ids
 *   jagged layout   offsets[0]=0, monotone, offsets[end]=sum(lengths)=|values|
 * Parity unpinned: the hash VALUES of SigridHash/NGram for composed inputs
 * other than the M=2^62 / SplitMix64 case rest on the DESIGN.md reading R1
 * (the paper names no hash function, L452) — DESIGN.md §4.
 */
#include "rap_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------ */
/* Hash primitive (reading R1): H(x) = first output of SplitMix64
 * seeded with x, i.e. mix(x + golden-gamma).  All arithmetic mod 2^64. */
uint64_t orc_H(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

/* Reading R2: range reduction floor(h * M / 2^64), result in [0, M). */
uint64_t orc_reduce(uint64_t h, int64_t M) {
  unsigned __int128 p = (unsigned __int128)h * (unsigned __int128)(uint64_t)M;
  return (uint64_t)(p >> 64);
}

/* SigridHash: "Compute hash value to normalize list of sparse
 * features".  Reading R3: reduce(H(H(u64(salt)) ^ u64(x)), M). */
int64_t orc_sigridhash(int64_t x, uint64_t salt, int64_t M) {
  uint64_t h = orc_H(orc_H(salt) ^ (uint64_t)x);
  return (int64_t)orc_reduce(h, M);
}

/* Logit: "Logit transform for normalization".  Reading R11
 * (torch.logit(x, eps) on f32): lo = eps, hi = 1 - eps in f32; clamp without
 * eating NaN; y = log(z / (1 - z)).  The quotient is the f32 IEEE quotient;
 * the logarithm is evaluated in fp64 and rounded once to f32. */
float orc_logit(float x, float eps) {
  float lo = eps;
  float hi = 1.0f - eps;
  float z = x;
  if (x < lo) z = lo;
  else if (x > hi) z = hi;
  float one_minus = 1.0f - z;
  float r = z / one_minus;
  return (float)log((double)r);
}

/* BoxCox: "BoxCox transform for normalization".  Reading R12
 * (scipy.special.boxcox): lambda == 0 -> log(x); otherwise
 * expm1(lambda * log(x)) / lambda, each step rounded to f32 (transcendentals
 * evaluated in fp64 and rounded once). */
float orc_boxcox(float x, float lambda) {
  if (lambda == 0.0f) return (float)log((double)x);
  float t = (float)log((double)x);
  float u = lambda * t;
  float e = (float)expm1((double)u);
  return e / lambda;
}

/* Bucketize: "Shard features based on bucket borders".
 * Reading R4: y = #{ i : borders[i] <= x } (x equal to a border goes to the
 * upper bucket; NaN compares false everywhere and lands in bucket 0). */
int64_t orc_bucketize_f(float x, const float* borders, int32_t m) {
  int64_t count = 0;
  for (int32_t i = 0; i < m; ++i)
    if (borders[i] <= x) count += 1;
  return count;
}

int64_t orc_bucketize_i(int64_t x, const int64_t* borders, int32_t m) {
  int64_t count = 0;
  for (int32_t i = 0; i < m; ++i)
    if (borders[i] <= x) count += 1;
  return count;
}

/* NGram, PAPER.md L459 ("Compute an n-gram between multiple sparse features")
 * and footnote L181-182 ("computes an n-gram across multiple sparse features to
 * generate new input features").  Reading R7: c = concatenation of the source
 * lists; one output per window start j = 0 .. len(c)-n (none if len(c) < n):
 *   h = H(salt); for i < n: h = H(h ^ c[j+i]); out_j = reduce(h, M).
 * Returns the number of outputs written. */
int64_t orc_ngram(const int64_t* c, int64_t len, int32_t n, uint64_t salt, int64_t M, int64_t* out) {
  int64_t count = len - (int64_t)n + 1;
  if (count < 0) count = 0;
  for (int64_t j = 0; j < count; ++j) {
    uint64_t h = orc_H(salt);
    for (int32_t i = 0; i < n; ++i) h = orc_H(h ^ (uint64_t)c[j + i]);
    out[j] = (int64_t)orc_reduce(h, M);
  }
  return count;
}

/* MapId: "Maps feature IDs to fixed values".  Reading R8: exact
 * match against the key table (linear scan), default when absent. */
static int64_t orc_mapid(int64_t x, const orc_node* nd) {
  for (int64_t i = 0; i < nd->map_size; ++i)
    if (nd->map_keys[i] == x) return nd->map_vals[i];
  return nd->map_default;
}

/* Clamp: "Clamp the sparse input based on the upper and lower
 * bound".  Reading R6: min(max(v, lo), hi) on int64 ids. */
static int64_t orc_clamp(int64_t v, int64_t lo, int64_t hi) {
  if (v < lo) v = lo;
  if (v > hi) v = hi;
  return v;
}

/* ------------------------------------------------------------------------ */
/* Per-row values flowing on DAG edges (DESIGN.md §3 "type system"). */
enum { T_NONE = 0, T_DENSE = 1, T_IDS = 2, T_VEC = 3 };

typedef struct {
  int type;
  float f;         /* T_DENSE: the value, NaN = null */
  int valid;       /* T_IDS: 0 = null list */
  int64_t len, cap;
  int64_t* ids;    /* T_IDS */
  int32_t k;       /* T_VEC width */
  float* vec;      /* T_VEC */
} rowval;

static int ids_reserve(rowval* v, int64_t want) {
  if (want <= v->cap) return 1;
  int64_t cap = v->cap ? v->cap : 16;
  while (cap < want) cap *= 2;
  int64_t* p = (int64_t*)realloc(v->ids, (size_t)cap * sizeof(int64_t));
  if (!p) return 0;
  v->ids = p;
  v->cap = cap;
  return 1;
}

static int bit_valid(const uint32_t* bm, int64_t b) {
  if (!bm) return 1;
  return (int)((bm[b >> 5] >> (b & 31)) & 1u);
}

/* ------------------------------------------------------------------------ */
/* Validation (DESIGN.md §3 "type system and validation"). */

static int input_type(const orc_graph* g, const int* node_type, int kind, int idx) {
  if (kind == ORC_IN_DENSE) return T_DENSE;
  if (kind == ORC_IN_SPARSE) return T_IDS;
  return node_type[idx];
}

/* Depth-first search for a cycle; state 0 = new, 1 = on stack, 2 = done. */
static int dfs_order(const orc_graph* g, int v, int* state, int* order, int* n_order) {
  if (state[v] == 2) return 1;
  if (state[v] == 1) return 0;
  state[v] = 1;
  const orc_node* nd = &g->nodes[v];
  for (int i = 0; i < nd->n_in; ++i)
    if (nd->in_kind[i] == ORC_IN_NODE)
      if (!dfs_order(g, nd->in_idx[i], state, order, n_order)) return 0;
  state[v] = 2;
  order[(*n_order)++] = v;
  return 1;
}

static int check_structure(const orc_graph* g) {
  for (int v = 0; v < g->n_nodes; ++v) {
    const orc_node* nd = &g->nodes[v];
    if (nd->op < ORC_FILLNULL || nd->op > ORC_MAPID) return ORC_ERR_INVALID_GRAPH;
    if (nd->op == ORC_NGRAM) {
      if (nd->n_in < 1 || nd->n_in > ORC_MAX_IN) return ORC_ERR_INVALID_PARAM;
    } else if (nd->n_in != 1) {
      return ORC_ERR_INVALID_GRAPH;
    }
    for (int i = 0; i < nd->n_in; ++i) {
      int kind = nd->in_kind[i], idx = nd->in_idx[i];
      if (kind == ORC_IN_NODE && (idx < 0 || idx >= g->n_nodes)) return ORC_ERR_INVALID_GRAPH;
      if (kind == ORC_IN_DENSE && (idx < 0 || idx >= g->n_dense)) return ORC_ERR_INVALID_GRAPH;
      if (kind == ORC_IN_SPARSE && (idx < 0 || idx >= g->n_sparse)) return ORC_ERR_INVALID_GRAPH;
      if (kind != ORC_IN_NODE && kind != ORC_IN_DENSE && kind != ORC_IN_SPARSE) return ORC_ERR_INVALID_GRAPH;
    }
  }
  for (int o = 0; o < g->n_outputs; ++o)
    if (g->outputs[o] < 0 || g->outputs[o] >= g->n_nodes) return ORC_ERR_INVALID_GRAPH;
  return ORC_OK;
}

/* Result type of node v given its (already typed) inputs; T_NONE = mismatch. */
static int node_type_of(const orc_graph* g, const int* node_type, int v) {
  const orc_node* nd = &g->nodes[v];
  int t0 = input_type(g, node_type, nd->in_kind[0], nd->in_idx[0]);
  switch (nd->op) {
    case ORC_FILLNULL:
      return (t0 == T_DENSE || t0 == T_IDS) ? t0 : T_NONE;
    case ORC_LOGIT:
    case ORC_BOXCOX:
      return t0 == T_DENSE ? T_DENSE : T_NONE;
    case ORC_BUCKETIZE:
      return (t0 == T_DENSE || t0 == T_IDS) ? T_IDS : T_NONE;
    case ORC_ONEHOT:
      return t0 == T_IDS ? T_VEC : T_NONE;
    case ORC_SIGRIDHASH:
    case ORC_FIRSTX:
    case ORC_CLAMP:
    case ORC_MAPID:
      return t0 == T_IDS ? T_IDS : T_NONE;
    case ORC_NGRAM:
      for (int i = 0; i < nd->n_in; ++i)
        if (input_type(g, node_type, nd->in_kind[i], nd->in_idx[i]) != T_IDS) return T_NONE;
      return T_IDS;
  }
  return T_NONE;
}

static int check_params(const orc_graph* g, const int* node_type) {
  for (int v = 0; v < g->n_nodes; ++v) {
    const orc_node* nd = &g->nodes[v];
    int t0 = input_type(g, node_type, nd->in_kind[0], nd->in_idx[0]);
    switch (nd->op) {
      case ORC_FILLNULL:
        if (t0 == T_DENSE && isnan(nd->f_fill)) return ORC_ERR_INVALID_PARAM;
        break;
      case ORC_LOGIT:
        if (!(nd->eps > 0.0f && nd->eps < 0.5f)) return ORC_ERR_INVALID_PARAM;
        break;
      case ORC_BOXCOX:
        if (!isfinite(nd->lambda)) return ORC_ERR_INVALID_PARAM;
        break;
      case ORC_BUCKETIZE:
        if (nd->n_borders < 1 || nd->n_borders > 65536) return ORC_ERR_INVALID_PARAM;
        if (t0 == T_DENSE) {
          if (!nd->f_borders) return ORC_ERR_INVALID_PARAM;
          for (int i = 0; i < nd->n_borders; ++i) {
            if (isnan(nd->f_borders[i])) return ORC_ERR_INVALID_PARAM;
            if (i > 0 && nd->f_borders[i] < nd->f_borders[i - 1]) return ORC_ERR_INVALID_PARAM;
          }
        } else {
          if (!nd->i_borders) return ORC_ERR_INVALID_PARAM;
          for (int i = 1; i < nd->n_borders; ++i)
            if (nd->i_borders[i] < nd->i_borders[i - 1]) return ORC_ERR_INVALID_PARAM;
        }
        break;
      case ORC_ONEHOT:
        if (nd->k_width < 1 || nd->k_width > 4096) return ORC_ERR_INVALID_PARAM;
        break;
      case ORC_SIGRIDHASH:
        if (nd->max_value < 1) return ORC_ERR_INVALID_PARAM;
        break;
      case ORC_FIRSTX:
        if (nd->x < 0) return ORC_ERR_INVALID_PARAM;
        break;
      case ORC_CLAMP:
        if (nd->lo > nd->hi) return ORC_ERR_INVALID_PARAM;
        break;
      case ORC_NGRAM:
        if (nd->n < 1 || nd->n > 8 || nd->max_value < 1) return ORC_ERR_INVALID_PARAM;
        break;
      case ORC_MAPID:
        if (nd->map_size < 0) return ORC_ERR_INVALID_PARAM;
        if (nd->map_size > 0 && (!nd->map_keys || !nd->map_vals)) return ORC_ERR_INVALID_PARAM;
        for (int64_t i = 0; i < nd->map_size; ++i)
          for (int64_t j = i + 1; j < nd->map_size; ++j)
            if (nd->map_keys[i] == nd->map_keys[j]) return ORC_ERR_INVALID_PARAM;
        break;
    }
  }
  return ORC_OK;
}

/* Validates g; on success fills node types + topological order (if given). */
static int validate(const orc_graph* g, int* node_type, int* order, int64_t* d_out, int64_t* f_out) {
  if (!g) return ORC_ERR_INVALID_ARGUMENT;
  if (g->n_dense < 0 || g->n_sparse < 0 || g->n_nodes < 0 || g->n_outputs < 0) return ORC_ERR_INVALID_ARGUMENT;
  if ((g->n_nodes > 0 && !g->nodes) || (g->n_outputs > 0 && !g->outputs)) return ORC_ERR_INVALID_ARGUMENT;
  int st = check_structure(g);
  if (st != ORC_OK) return st;
  int* state = (int*)calloc((size_t)g->n_nodes + 1, sizeof(int));
  if (!state) return ORC_ERR_NOMEM;
  int n_order = 0;
  for (int v = 0; v < g->n_nodes; ++v) {
    if (!dfs_order(g, v, state, order, &n_order)) {
      free(state);
      return ORC_ERR_INVALID_GRAPH;
    }
  }
  free(state);
  for (int i = 0; i < n_order; ++i) {
    int v = order[i];
    node_type[v] = node_type_of(g, node_type, v);
    if (node_type[v] == T_NONE) return ORC_ERR_INVALID_GRAPH;
  }
  st = check_params(g, node_type);
  if (st != ORC_OK) return st;
  int64_t d = 0, f = 0;
  for (int o = 0; o < g->n_outputs; ++o) {
    int t = node_type[g->outputs[o]];
    if (t == T_DENSE) d += 1;
    else if (t == T_VEC) d += g->nodes[g->outputs[o]].k_width;
    else f += 1;
  }
  if (d_out) *d_out = d;
  if (f_out) *f_out = f;
  return ORC_OK;
}

int orc_validate(const orc_graph* g, int64_t* d_out, int64_t* f_out) {
  if (!g) return ORC_ERR_INVALID_ARGUMENT;
  int n = g->n_nodes > 0 ? g->n_nodes : 1;
  int* node_type = (int*)calloc((size_t)n, sizeof(int));
  int* order = (int*)calloc((size_t)n, sizeof(int));
  int st = (node_type && order) ? validate(g, node_type, order, d_out, f_out) : ORC_ERR_NOMEM;
  free(node_type);
  free(order);
  return st;
}

/* ------------------------------------------------------------------------ */
/* Evaluation of one node on one row. */

/* Fetch an input of node nd for row b: raw columns are materialised into
 * `scratch`, node inputs point at their already-evaluated row value. */
static const rowval* fetch_input(const orc_graph* g, const orc_batch* bt, const rowval* vals, int kind,
                                 int idx, int64_t b, rowval* scratch) {
  if (kind == ORC_IN_NODE) return &vals[idx];
  if (kind == ORC_IN_DENSE) {
    /* Reading R14: a null dense slot is NaN downstream. */
    scratch->type = T_DENSE;
    scratch->f = bit_valid(bt->dense_valid ? bt->dense_valid[idx] : NULL, b) ? bt->dense[idx][b] : NAN;
    return scratch;
  }
  /* Raw sparse column: Arrow list<int64>; a null row is a null list whatever
   * its child segment holds (reading R14). */
  scratch->type = T_IDS;
  scratch->valid = bit_valid(bt->sp_valid ? bt->sp_valid[idx] : NULL, b);
  scratch->len = 0;
  if (scratch->valid) {
    int64_t s = bt->sp_off[idx][b], e = bt->sp_off[idx][b + 1];
    int64_t L = e - s;
    if (!ids_reserve(scratch, L)) return NULL;
    for (int64_t j = 0; j < L; ++j) scratch->ids[j] = bt->sp_val[idx][s + j];
    scratch->len = L;
  }
  return scratch;
}

static int eval_node(const orc_graph* g, const orc_batch* bt, rowval* vals, int v, int64_t b, rowval* scratch) {
  const orc_node* nd = &g->nodes[v];
  rowval* out = &vals[v];
  const rowval* in0 = fetch_input(g, bt, vals, nd->in_kind[0], nd->in_idx[0], b, &scratch[0]);
  if (!in0) return 0;
  switch (nd->op) {
    case ORC_FILLNULL:
      /* PAPER.md L462 "Fill NA/NaN values using the specified value".
       * Reading R10: dense NaN (null or NaN payload) -> f_fill; a null list ->
       * the one-element list [i_fill]; a valid (possibly empty) list unchanged. */
      if (in0->type == T_DENSE) {
        out->type = T_DENSE;
        out->f = isnan(in0->f) ? nd->f_fill : in0->f;
      } else {
        out->type = T_IDS;
        if (!in0->valid) {
          if (!ids_reserve(out, 1)) return 0;
          out->valid = 1;
          out->len = 1;
          out->ids[0] = nd->i_fill;
        } else {
          if (!ids_reserve(out, in0->len)) return 0;
          out->valid = 1;
          out->len = in0->len;
          for (int64_t j = 0; j < in0->len; ++j) out->ids[j] = in0->ids[j];
        }
      }
      return 1;
    case ORC_LOGIT:
      out->type = T_DENSE;
      out->f = orc_logit(in0->f, nd->eps);
      return 1;
    case ORC_BOXCOX:
      out->type = T_DENSE;
      out->f = orc_boxcox(in0->f, nd->lambda);
      return 1;
    case ORC_BUCKETIZE:
      out->type = T_IDS;
      if (in0->type == T_DENSE) {
        /* A dense scalar becomes a length-1 id list (feature generation, L457-458). */
        if (!ids_reserve(out, 1)) return 0;
        out->valid = 1;
        out->len = 1;
        out->ids[0] = orc_bucketize_f(in0->f, nd->f_borders, nd->n_borders);
      } else {
        if (!ids_reserve(out, in0->len)) return 0;
        out->valid = in0->valid;
        out->len = in0->valid ? in0->len : 0;
        for (int64_t j = 0; j < out->len; ++j) out->ids[j] = orc_bucketize_i(in0->ids[j], nd->i_borders, nd->n_borders);
      }
      return 1;
    case ORC_ONEHOT:
      /* PAPER.md L449 "Apply one hot encoding".  Reading R9: K f32 columns,
       * column k = 1 if some id equals k; out-of-range ids ignored; a null or
       * empty list gives all zeros. */
      out->type = T_VEC;
      out->k = nd->k_width;
      if (!out->vec) {
        out->vec = (float*)malloc((size_t)nd->k_width * sizeof(float));
        if (!out->vec) return 0;
      }
      for (int32_t k = 0; k < nd->k_width; ++k) out->vec[k] = 0.0f;
      if (in0->valid)
        for (int64_t j = 0; j < in0->len; ++j)
          if (in0->ids[j] >= 0 && in0->ids[j] < nd->k_width) out->vec[in0->ids[j]] = 1.0f;
      return 1;
    case ORC_SIGRIDHASH:
    case ORC_CLAMP:
    case ORC_MAPID:
      out->type = T_IDS;
      if (!ids_reserve(out, in0->len)) return 0;
      out->valid = in0->valid;
      out->len = in0->valid ? in0->len : 0;
      for (int64_t j = 0; j < out->len; ++j) {
        int64_t x = in0->ids[j];
        if (nd->op == ORC_SIGRIDHASH) out->ids[j] = orc_sigridhash(x, nd->salt, nd->max_value);
        else if (nd->op == ORC_CLAMP) out->ids[j] = orc_clamp(x, nd->lo, nd->hi);
        else out->ids[j] = orc_mapid(x, nd);
      }
      return 1;
    case ORC_FIRSTX: {
      /* PAPER.md L454 "List truncation".  Reading R5: first min(L, x) ids. */
      out->type = T_IDS;
      out->valid = in0->valid;
      int64_t L = in0->valid ? in0->len : 0;
      int64_t keep = L < nd->x ? L : nd->x;
      if (!ids_reserve(out, keep)) return 0;
      for (int64_t j = 0; j < keep; ++j) out->ids[j] = in0->ids[j];
      out->len = keep;
      return 1;
    }
    case ORC_NGRAM: {
      /* Concatenate the k source lists (a null source contributes nothing). */
      rowval* cat = &scratch[ORC_MAX_IN];
      cat->len = 0;
      for (int i = 0; i < nd->n_in; ++i) {
        const rowval* src = fetch_input(g, bt, vals, nd->in_kind[i], nd->in_idx[i], b, &scratch[i]);
        if (!src) return 0;
        if (!src->valid) continue;
        if (!ids_reserve(cat, cat->len + src->len)) return 0;
        for (int64_t j = 0; j < src->len; ++j) cat->ids[cat->len + j] = src->ids[j];
        cat->len += src->len;
      }
      out->type = T_IDS;
      out->valid = 1;
      int64_t cnt = cat->len - nd->n + 1;
      if (!ids_reserve(out, cnt > 0 ? cnt : 0)) return 0;
      out->len = orc_ngram(cat->ids, cat->len, nd->n, nd->salt, nd->max_value, out->ids);
      return 1;
    }
  }
  return 0;
}

/* ------------------------------------------------------------------------ */

typedef struct {
  int64_t len, cap;
  int64_t* v;
} grow64;

static int grow_push(grow64* a, const int64_t* src, int64_t n) {
  if (a->len + n > a->cap) {
    int64_t cap = a->cap ? a->cap : 1024;
    while (cap < a->len + n) cap *= 2;
    int64_t* p = (int64_t*)realloc(a->v, (size_t)cap * sizeof(int64_t));
    if (!p) return 0;
    a->v = p;
    a->cap = cap;
  }
  for (int64_t j = 0; j < n; ++j) a->v[a->len + j] = src[j];
  a->len += n;
  return 1;
}

int orc_run(const orc_graph* g, const orc_batch* bt, orc_result* r) {
  if (!g || !bt || !r) return ORC_ERR_INVALID_ARGUMENT;
  memset(r, 0, sizeof(*r));
  if (bt->n_rows < 0) return ORC_ERR_INVALID_ARGUMENT;
  int n = g->n_nodes > 0 ? g->n_nodes : 1;
  int* node_type = (int*)calloc((size_t)n, sizeof(int));
  int* order = (int*)calloc((size_t)n, sizeof(int));
  if (!node_type || !order) {
    free(node_type);
    free(order);
    return ORC_ERR_NOMEM;
  }
  int64_t d_out = 0, f_out = 0;
  int st = validate(g, node_type, order, &d_out, &f_out);
  if (st != ORC_OK) {
    free(node_type);
    free(order);
    return st;
  }
  const int64_t B = bt->n_rows;
  rowval* vals = (rowval*)calloc((size_t)n, sizeof(rowval));
  rowval scratch[ORC_MAX_IN + 1];
  memset(scratch, 0, sizeof(scratch));
  grow64* feat = (grow64*)calloc((size_t)(f_out > 0 ? f_out : 1), sizeof(grow64));
  r->n_rows = B;
  r->d_out = d_out;
  r->f_out = f_out;
  r->dense = (float*)malloc((size_t)(B * d_out > 0 ? B * d_out : 1) * sizeof(float));
  r->lengths = (int32_t*)malloc((size_t)(B * f_out > 0 ? B * f_out : 1) * sizeof(int32_t));
  r->offsets = (int64_t*)malloc((size_t)(B * f_out + 1) * sizeof(int64_t));
  int ok = vals && feat && r->dense && r->lengths && r->offsets;

  /* Row by row: evaluate every node in topological order, then emit. */
  for (int64_t b = 0; ok && b < B; ++b) {
    for (int i = 0; ok && i < g->n_nodes; ++i) ok = eval_node(g, bt, vals, order[i], b, scratch);
    int64_t col = 0, f = 0;
    for (int o = 0; ok && o < g->n_outputs; ++o) {
      const rowval* v = &vals[g->outputs[o]];
      if (v->type == T_DENSE) {
        r->dense[b * d_out + col] = v->f;
        col += 1;
      } else if (v->type == T_VEC) {
        for (int32_t k = 0; k < v->k; ++k) r->dense[b * d_out + col + k] = v->vec[k];
        col += v->k;
      } else {
        /* Reading R14: a null list is emitted with length 0. */
        int64_t L = v->valid ? v->len : 0;
        r->lengths[f * B + b] = (int32_t)L;
        ok = grow_push(&feat[f], v->ids, L);
        f += 1;
      }
    }
  }
  /* Feature-major jagged layout (reading R17): offsets = exclusive scan of the
   * flattened lengths; values concatenated in (feature, row, element) order. */
  int64_t total = 0;
  if (ok) {
    r->offsets[0] = 0;
    for (int64_t i = 0; i < B * f_out; ++i) r->offsets[i + 1] = r->offsets[i] + r->lengths[i];
    for (int64_t f = 0; f < f_out; ++f) total += feat[f].len;
    r->values = (int64_t*)malloc((size_t)(total > 0 ? total : 1) * sizeof(int64_t));
    ok = r->values != NULL;
  }
  if (ok) {
    int64_t pos = 0;
    for (int64_t f = 0; f < f_out; ++f) {
      for (int64_t j = 0; j < feat[f].len; ++j) r->values[pos + j] = feat[f].v[j];
      pos += feat[f].len;
    }
    r->n_values = total;
  }
  for (int i = 0; vals && i < n; ++i) {
    free(vals[i].ids);
    free(vals[i].vec);
  }
  for (int i = 0; i <= ORC_MAX_IN; ++i) free(scratch[i].ids);
  for (int64_t f = 0; feat && f < f_out; ++f) free(feat[f].v);
  free(feat);
  free(vals);
  free(node_type);
  free(order);
  if (!ok) {
    orc_free(r);
    return ORC_ERR_NOMEM;
  }
  return ORC_OK;
}

void orc_free(orc_result* r) {
  if (!r) return;
  free(r->dense);
  free(r->lengths);
  free(r->offsets);
  free(r->values);
  r->dense = NULL;
  r->lengths = NULL;
  r->offsets = NULL;
  r->values = NULL;
}
