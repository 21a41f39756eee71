// rap_plan.cpp — host planner and C ABI (include/rap.h).
//
// rap_plan_create = row a0 of DESIGN.md §1: validate the preprocessing DAG
// with the R20 checks, lower every output to a device op
// program (rap_internal.h), precompute H(salt) and sorted MapId / Bucketize
// tables, size the (feature, row-range) descriptor geometry and the grid from
// the SM budget (resource-aware sharding, L1351-1366 §6.2).  rap_preprocess
// = row a1: one launch, no host sync.
#include <cuda.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <limits>
#include <map>
#include <mutex>
#include <numeric>
#include <string>
#include <utility>
#include <vector>

#include "../../include/rap.h"
#include "rap_internal.h"

using namespace rapk;

namespace {

thread_local std::string g_last_error;

rap_status fail(rap_status s, const std::string& msg) {
  g_last_error = msg;
  return s;
}

rap_status cuda_fail(cudaError_t e, const char* what) {
  return fail(RAP_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

// Node value types (DESIGN.md §3 "type system").
enum VType { VT_NONE = 0, VT_DENSE = 1, VT_IDS = 2, VT_VEC = 3 };

// Host-only intermediate form of the lowering (the device sees SProg / DProg).
struct DenseExpr {
  int32_t col, op_begin, op_end, pad;
};
enum HUnitKind { HU_DENSE = 0, HU_ONEHOT = 1 };
struct Unit {  // one dense output: a Dense node (idx = dense expr) or a OneHot (idx = chain)
  int32_t kind, idx, col, width;
};
struct SparseOut {
  int32_t chain, rows_per_desc;
};

int64_t sat_add(int64_t a, int64_t b) {
  if (a > INT64_MAX - b) return INT64_MAX;
  return a + b;
}
int64_t sat_mul(int64_t a, int64_t b) {
  if (a != 0 && b > INT64_MAX / a) return INT64_MAX;
  return a * b;
}

}  // namespace

// Latency-model constants (rap_predict_latency_us): t0/c per kernel family
// and the HBM bandwidth, fitted on B200 (profiles/r02b_cost_model_fit.txt).
#ifndef RAP_MODEL_FIT
#define RAP_MODEL_FIT 28.5241, 1.99159e-05, 0, 0, 12.1317, 0, 0.0101896, 0, 12.4147, 0, 0.003001, 0, 6446.6
#endif

struct rap_plan {
  int device = 0, sm_count = 0, budget = 0, ctas_per_sm = 1, smem = 0;
  int n_dense_in = 0, n_sparse_in = 0;
  int rank = 0, world = 1;  // sharded plan: dense outputs cover rap_shard_rows(rank, world)
  // lowered program (host copies)
  std::vector<DevOp> ops;
  std::vector<DenseExpr> dexprs;
  std::vector<Chain> chains;
  std::vector<NGramDesc> ngrams;
  std::vector<SparseOut> souts;
  std::vector<float> ftab;
  std::vector<int64_t> itab;
  std::vector<int> used_dense, used_sparse;
  // flattened device programs
  std::vector<SProg> sprogs, oprogs;
  std::vector<DProg> dprogs;
  int d_out = 0, rows_dense = 256;
  // device program blob
  unsigned char* blob = nullptr;
  size_t off_ops = 0, off_sprogs = 0, off_oprogs = 0, off_dprogs = 0, off_ftab = 0, off_itab = 0;
  // per-CTA partition of the unit sequence (cost model),
  // re-uploaded only when its key (rows, grid, quantised list lengths) changes
  // kPartSlots cached partitions (batches of different shapes alternate
  // without re-uploads); slot i: key part_keys[i], device d_part + i * kPartLen
  std::vector<std::vector<int64_t>> part_keys;
  std::vector<char> part_pin;  // slot used by a launch captured into a CUDA graph: never evicted
  int part_next = 0;
  int64_t* d_part = nullptr;               // [kPartSlots * kPartLen]
  int64_t* h_part = nullptr;               // pinned staging, same layout
  // scheduling state
  unsigned long long* d_sched = nullptr;   // CTAs done, launch epoch, rank counter
  unsigned long long* d_agg = nullptr;     // [kMaxCtas] per-rank aggregate words
  int32_t* d_err = nullptr;
  int64_t n_launches = 0;
  int64_t last_n_desc = 0;
  // profiling aid (rap_debug_trace)
  unsigned long long* d_trace = nullptr;
  int64_t trace_cap = 0;
  // host-buffer staging (rap_preprocess_host)
  std::vector<void*> stage;
  std::vector<size_t> stage_cap;
  int64_t partition_uploads = 0;
  // row-block kernel (rap_rows.cu)
  int kernel_mode = RAP_KERNEL_AUTO, kernel_last = 0;
  int rb_fits = 0, rb_ctas_per_sm = 0, rb_smem = 0, rb_max_fl = 0, rb_max_cols = 0, rb_n_memo = 0;
  int rb_last_grid = 0;  // CTAs of the last row-block / generated launch
  int rb_dense_bytes = 0;
  unsigned long long rb_all_cols = 0;  // raw sparse columns the sparse outputs read
  std::vector<RbFeat> rbfeat;     // by output index
  std::vector<int32_t> rb_perm;   // processing order
  size_t off_rbfeat = 0, off_perm = 0;
  unsigned long long* d_agg_rb = nullptr;  // [n_sparse_out][n_rb] row-block totals, then [n_sparse_out] totals
  int rb_last_n_rb = 0, rb_last_n_fg = 0, rb_last_rows = 0;
  // plan-specialised row-block kernel (rap_jit.cpp), built on first use
  JitModule* jit[4] = {nullptr, nullptr, nullptr, nullptr};  // [small | int32 values << 1] variants
  int jit_state = 0, jit_ctas_per_sm = 0;  // state of the last variant asked for
  int jit_st[4] = {0, 0, 0, 0}, jit_occ[4] = {0, 0, 0, 0};
  int jit_smem = 0, jit_dense_bytes = 0, jit_id_slots = 0, jit_tab_bytes = 0;
  int jit_max_fl = 0;  // the generated kernel's one group: every output (<= kJitMaxF)
  double jit_s = 0;
};

namespace {

// ----------------------------------------------------------------------------
// Validation (R20).  Mirrors the oracle's order; implemented independently.
struct Validated {
  std::vector<int> type;   // per node
  std::vector<int> order;  // topological
  int64_t d_out = 0, f_out = 0;
};

int in_type(const rap_graph* g, const std::vector<int>& type, int32_t ref) {
  if (ref >= 0) return type[ref];
  if ((-ref) % 2 == 1) return VT_DENSE;  // -1 - 2c
  return VT_IDS;                          // -2 - 2c
}

bool ref_ok(const rap_graph* g, int32_t ref) {
  if (ref >= 0) return ref < g->n_nodes;
  int32_t m = -ref;
  if (m % 2 == 1) {
    int c = (m - 1) / 2;
    return c < g->n_dense_in;
  }
  int c = (m - 2) / 2;
  return c < g->n_sparse_in;
}

rap_status validate(const rap_graph* g, const rap_op_param* params, int32_t n_params, Validated* v) {
  if (!g) return fail(RAP_ERR_INVALID_ARGUMENT, "graph is NULL");
  if (g->n_dense_in < 0 || g->n_sparse_in < 0 || g->n_nodes < 0 || g->n_outputs < 0)
    return fail(RAP_ERR_INVALID_ARGUMENT, "negative count in graph");
  if ((g->n_nodes > 0 && !g->nodes) || (g->n_outputs > 0 && !g->output_nodes))
    return fail(RAP_ERR_INVALID_ARGUMENT, "graph arrays are NULL");
  if (n_params < 0 || (n_params > 0 && !params)) return fail(RAP_ERR_INVALID_ARGUMENT, "params array");
  const int N = g->n_nodes;
  for (int i = 0; i < N; ++i) {
    const rap_node& nd = g->nodes[i];
    if (nd.param < 0 || nd.param >= n_params)
      return fail(RAP_ERR_INVALID_ARGUMENT, "node " + std::to_string(i) + ": param index out of range");
  }
  for (int i = 0; i < N; ++i) {
    const rap_node& nd = g->nodes[i];
    if (nd.op < RAP_OP_FILLNULL || nd.op > RAP_OP_MAPID)
      return fail(RAP_ERR_INVALID_GRAPH, "node " + std::to_string(i) + ": unknown op");
    if (nd.op == RAP_OP_NGRAM) {
      if (nd.n_inputs < 1 || nd.n_inputs > kMaxNgramK)
        return fail(RAP_ERR_INVALID_PARAM, "node " + std::to_string(i) + ": NGram needs 1..8 inputs");
    } else if (nd.n_inputs != 1) {
      return fail(RAP_ERR_INVALID_GRAPH, "node " + std::to_string(i) + ": op takes one input");
    }
    if (!nd.inputs) return fail(RAP_ERR_INVALID_ARGUMENT, "node inputs NULL");
    for (int k = 0; k < nd.n_inputs; ++k)
      if (!ref_ok(g, nd.inputs[k]))
        return fail(RAP_ERR_INVALID_GRAPH, "node " + std::to_string(i) + ": input reference out of range");
  }
  for (int o = 0; o < g->n_outputs; ++o)
    if (g->output_nodes[o] < 0 || g->output_nodes[o] >= N)
      return fail(RAP_ERR_INVALID_GRAPH, "output reference out of range");
  // cycle check + topological order (iterative DFS)
  std::vector<int> state(N, 0);
  v->order.clear();
  for (int s = 0; s < N; ++s) {
    if (state[s]) continue;
    std::vector<std::pair<int, int>> st{{s, 0}};
    state[s] = 1;
    while (!st.empty()) {
      auto& top = st.back();
      const rap_node& nd = g->nodes[top.first];
      if (top.second < nd.n_inputs) {
        int32_t ref = nd.inputs[top.second++];
        if (ref >= 0) {
          if (state[ref] == 1) return fail(RAP_ERR_INVALID_GRAPH, "cycle in preprocessing graph");
          if (state[ref] == 0) {
            state[ref] = 1;
            st.push_back({ref, 0});
          }
        }
      } else {
        state[top.first] = 2;
        v->order.push_back(top.first);
        st.pop_back();
      }
    }
  }
  v->type.assign(N, VT_NONE);
  for (int i : v->order) {
    const rap_node& nd = g->nodes[i];
    int t0 = in_type(g, v->type, nd.inputs[0]);
    int t = VT_NONE;
    switch (nd.op) {
      case RAP_OP_FILLNULL: t = (t0 == VT_DENSE || t0 == VT_IDS) ? t0 : VT_NONE; break;
      case RAP_OP_LOGIT:
      case RAP_OP_BOXCOX: t = t0 == VT_DENSE ? VT_DENSE : VT_NONE; break;
      case RAP_OP_BUCKETIZE: t = (t0 == VT_DENSE || t0 == VT_IDS) ? VT_IDS : VT_NONE; break;
      case RAP_OP_ONEHOT: t = t0 == VT_IDS ? VT_VEC : VT_NONE; break;
      case RAP_OP_NGRAM:
        t = VT_IDS;
        for (int k = 0; k < nd.n_inputs; ++k)
          if (in_type(g, v->type, nd.inputs[k]) != VT_IDS) t = VT_NONE;
        break;
      default: t = t0 == VT_IDS ? VT_IDS : VT_NONE; break;
    }
    if (t == VT_NONE) return fail(RAP_ERR_INVALID_GRAPH, "node " + std::to_string(i) + ": input type mismatch");
    v->type[i] = t;
  }
  for (int i = 0; i < N; ++i) {
    const rap_node& nd = g->nodes[i];
    const rap_op_param& pr = params[nd.param];
    const int t0 = in_type(g, v->type, nd.inputs[0]);
    const std::string who = "node " + std::to_string(i) + ": ";
    switch (nd.op) {
      case RAP_OP_FILLNULL:
        if (t0 == VT_DENSE && std::isnan(pr.f_fill)) return fail(RAP_ERR_INVALID_PARAM, who + "fill is NaN");
        break;
      case RAP_OP_LOGIT:
        if (!(pr.eps > 0.0f && pr.eps < 0.5f)) return fail(RAP_ERR_INVALID_PARAM, who + "eps not in (0, 0.5)");
        break;
      case RAP_OP_BOXCOX:
        if (!std::isfinite(pr.lambda)) return fail(RAP_ERR_INVALID_PARAM, who + "lambda not finite");
        break;
      case RAP_OP_BUCKETIZE:
        if (pr.n_borders < 1 || pr.n_borders > 65536) return fail(RAP_ERR_INVALID_PARAM, who + "borders count");
        if (!pr.borders) return fail(RAP_ERR_INVALID_PARAM, who + "borders NULL");
        if (t0 == VT_DENSE) {
          const float* b = static_cast<const float*>(pr.borders);
          for (int k = 0; k < pr.n_borders; ++k) {
            if (std::isnan(b[k])) return fail(RAP_ERR_INVALID_PARAM, who + "NaN border");
            if (k > 0 && b[k] < b[k - 1]) return fail(RAP_ERR_INVALID_PARAM, who + "borders not sorted");
          }
        } else {
          const int64_t* b = static_cast<const int64_t*>(pr.borders);
          for (int k = 1; k < pr.n_borders; ++k)
            if (b[k] < b[k - 1]) return fail(RAP_ERR_INVALID_PARAM, who + "borders not sorted");
        }
        break;
      case RAP_OP_ONEHOT:
        if (pr.k_width < 1 || pr.k_width > 4096) return fail(RAP_ERR_INVALID_PARAM, who + "K not in [1, 4096]");
        break;
      case RAP_OP_SIGRIDHASH:
        if (pr.max_value < 1) return fail(RAP_ERR_INVALID_PARAM, who + "max_value < 1");
        break;
      case RAP_OP_FIRSTX:
        if (pr.x < 0) return fail(RAP_ERR_INVALID_PARAM, who + "x < 0");
        break;
      case RAP_OP_CLAMP:
        if (pr.lo > pr.hi) return fail(RAP_ERR_INVALID_PARAM, who + "lo > hi");
        break;
      case RAP_OP_NGRAM:
        if (pr.n < 1 || pr.n > 8 || pr.max_value < 1) return fail(RAP_ERR_INVALID_PARAM, who + "n or max_value");
        break;
      case RAP_OP_MAPID: {
        if (pr.map_size < 0) return fail(RAP_ERR_INVALID_PARAM, who + "map_size < 0");
        if (pr.map_size > 0 && (!pr.map_keys || !pr.map_vals)) return fail(RAP_ERR_INVALID_PARAM, who + "map NULL");
        if (pr.map_size > (int64_t)INT32_MAX) return fail(RAP_ERR_INVALID_PARAM, who + "map too large");
        std::vector<int64_t> k(pr.map_keys, pr.map_keys + pr.map_size);
        std::sort(k.begin(), k.end());
        if (std::adjacent_find(k.begin(), k.end()) != k.end())
          return fail(RAP_ERR_INVALID_PARAM, who + "duplicate MapId key");
        break;
      }
    }
  }
  v->d_out = v->f_out = 0;
  for (int o = 0; o < g->n_outputs; ++o) {
    int t = v->type[g->output_nodes[o]];
    if (t == VT_DENSE) v->d_out += 1;
    else if (t == VT_VEC) v->d_out += params[g->nodes[g->output_nodes[o]].param].k_width;
    else v->f_out += 1;
  }
  return RAP_OK;
}

// ----------------------------------------------------------------------------
// Lowering.
struct Lowerer {
  const rap_graph* g;
  const rap_op_param* params;
  rap_plan* P;
  std::vector<int> dense_memo, chain_memo;

  int lower_dense(int32_t ref) {
    if (ref >= 0 && dense_memo[ref] >= 0) return dense_memo[ref];
    std::vector<int> path;  // node ids, output -> source
    int32_t cur = ref;
    while (cur >= 0) {
      path.push_back(cur);
      cur = g->nodes[cur].inputs[0];
    }
    const int col = (-cur - 1) / 2;
    DenseExpr de{};
    de.col = col;
    de.op_begin = (int)P->ops.size();
    for (auto it = path.rbegin(); it != path.rend(); ++it) {
      const rap_node& nd = g->nodes[*it];
      const rap_op_param& pr = params[nd.param];
      DevOp op{};
      if (nd.op == RAP_OP_FILLNULL) {
        op.kind = OK_FILL_F;
        op.f0 = pr.f_fill;
      } else if (nd.op == RAP_OP_LOGIT) {
        op.kind = OK_LOGIT;
        volatile float eps = pr.eps;
        op.f0 = eps;
        op.f1 = 1.0f - eps;  // f32 arithmetic (R11)
      } else {
        op.kind = OK_BOXCOX;
        op.f0 = pr.lambda;
      }
      P->ops.push_back(op);
    }
    de.op_end = (int)P->ops.size();
    P->dexprs.push_back(de);
    const int idx = (int)P->dexprs.size() - 1;
    if (ref >= 0) dense_memo[ref] = idx;
    return idx;
  }

  // returns chain index, or -1 with *st set
  int lower_ids(int32_t ref, bool allow_ngram, rap_status* st) {
    if (ref >= 0 && chain_memo[ref] >= 0) {
      const Chain& c = P->chains[chain_memo[ref]];
      if (c.src_kind == SRC_NGRAM && !allow_ngram) {
        *st = fail(RAP_ERR_UNSUPPORTED, "NGram over an NGram output is not supported");
        return -1;
      }
      return chain_memo[ref];
    }
    // walk back through single-input id ops
    std::vector<int> path;
    int32_t cur = ref;
    Chain ch{};
    ch.xcap = kNoCap;
    ch.null_xcap = kNoCap;
    while (true) {
      if (cur < 0) {  // raw sparse column
        ch.src_kind = SRC_SPARSE;
        ch.src = (-cur - 2) / 2;
        break;
      }
      const rap_node& nd = g->nodes[cur];
      if (nd.op == RAP_OP_NGRAM) {
        ch.src_kind = SRC_NGRAM;
        break;
      }
      if (nd.op == RAP_OP_BUCKETIZE && in_is_dense(nd.inputs[0])) {
        ch.src_kind = SRC_DENSE_BUCKET;
        break;
      }
      path.push_back(cur);
      cur = nd.inputs[0];
    }
    if (ch.src_kind == SRC_NGRAM) {
      if (!allow_ngram) {
        *st = fail(RAP_ERR_UNSUPPORTED, "NGram over an NGram output is not supported");
        return -1;
      }
      const rap_node& nd = g->nodes[cur];
      const rap_op_param& pr = params[nd.param];
      NGramDesc ng{};
      ng.n = pr.n;
      ng.k = nd.n_inputs;
      ng.hsalt = splitmix_H(pr.salt);
      ng.M = pr.max_value;
      for (int k = 0; k < nd.n_inputs; ++k) {
        int c = lower_ids(nd.inputs[k], false, st);
        if (c < 0) return -1;
        ng.chain[k] = c;
      }
      P->ngrams.push_back(ng);
      ch.src = (int)P->ngrams.size() - 1;
    } else if (ch.src_kind == SRC_DENSE_BUCKET) {
      const rap_node& nd = g->nodes[cur];
      const rap_op_param& pr = params[nd.param];
      const DenseExpr& de = P->dexprs[lower_dense(nd.inputs[0])];
      ch.src = de.col;  // raw dense column; its dense ops precede the bucketize
      ch.dop_begin = de.op_begin;
      ch.dop_end = de.op_end;
      ch.btab = (int)P->ftab.size();
      ch.bm = pr.n_borders;
      const float* b = static_cast<const float*>(pr.borders);
      P->ftab.insert(P->ftab.end(), b, b + pr.n_borders);
    }
    ch.op_begin = (int)P->ops.size();
    bool fill_seen = false;
    int null_begin = 0;
    for (auto it = path.rbegin(); it != path.rend(); ++it) {
      const rap_node& nd = g->nodes[*it];
      const rap_op_param& pr = params[nd.param];
      DevOp op{};
      switch (nd.op) {
        case RAP_OP_FILLNULL:
          if (!fill_seen && ch.src_kind == SRC_SPARSE) {
            fill_seen = true;
            ch.fill = pr.i_fill;
            null_begin = (int)P->ops.size();
          }
          continue;
        case RAP_OP_FIRSTX:
          ch.xcap = std::min(ch.xcap, pr.x);
          if (fill_seen) ch.null_xcap = std::min(ch.null_xcap, pr.x);
          continue;
        case RAP_OP_CLAMP:
          op.kind = OK_CLAMP;
          op.a = pr.lo;
          op.b = pr.hi;
          break;
        case RAP_OP_SIGRIDHASH:
          op.kind = OK_SIGRID;
          op.hsalt = splitmix_H(pr.salt);
          op.M = pr.max_value;
          break;
        case RAP_OP_BUCKETIZE: {
          op.kind = OK_BUCKET_I;
          op.a = (int64_t)P->itab.size();
          op.m = pr.n_borders;
          const int64_t* b = static_cast<const int64_t*>(pr.borders);
          P->itab.insert(P->itab.end(), b, b + pr.n_borders);
          break;
        }
        case RAP_OP_MAPID: {
          // open-addressing hash table: 2^lg slots, load <= 1/2, Fibonacci
          // hashing, linear probing; INT64_MIN marks an empty slot
          op.kind = OK_MAPID;
          op.b = pr.map_default;
          int lg = 4;
          while ((int64_t(1) << lg) < 2 * pr.map_size) ++lg;
          const int64_t cap = int64_t(1) << lg;
          if (P->itab.size() % 2) P->itab.push_back(0);  // 16-byte aligned slots
          op.a = (int64_t)P->itab.size();
          op.m = lg;
          P->itab.resize(P->itab.size() + 2 * cap, 0);
          int64_t* tab = P->itab.data() + op.a;
          for (int64_t k = 0; k < cap; ++k) tab[2 * k] = INT64_MIN;
          for (int64_t k = 0; k < pr.map_size; ++k) {
            const int64_t key = pr.map_keys[k];
            if (key == INT64_MIN) {
              op.M = 1;
              op.hsalt = (uint64_t)pr.map_vals[k];
              continue;
            }
            uint64_t i = ((uint64_t)key * 0x9E3779B97F4A7C15ull) >> (64 - lg);
            while (tab[2 * i] != INT64_MIN) i = (i + 1) & (uint64_t)(cap - 1);
            tab[2 * i] = key;
            tab[2 * i + 1] = pr.map_vals[k];
          }
          break;
        }
        default:
          *st = fail(RAP_ERR_UNSUPPORTED, "unexpected op in id chain");
          return -1;
      }
      P->ops.push_back(op);
    }
    ch.op_end = (int)P->ops.size();
    ch.has_fill = fill_seen ? 1 : 0;
    ch.null_op_begin = fill_seen ? null_begin : ch.op_end;
    P->chains.push_back(ch);
    const int idx = (int)P->chains.size() - 1;
    if (ref >= 0) chain_memo[ref] = idx;
    return idx;
  }

  bool in_is_dense(int32_t ref) {
    if (ref < 0) return (-ref) % 2 == 1;
    return type_of[ref] == VT_DENSE;
  }
  std::vector<int> type_of;
};

template <class T>
size_t push_blob(std::vector<unsigned char>& blob, const std::vector<T>& v) {
  size_t off = (blob.size() + 15) / 16 * 16;
  blob.resize(off + v.size() * sizeof(T));
  if (!v.empty()) memcpy(blob.data() + off, v.data(), v.size() * sizeof(T));
  return off;
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

int64_t chain_bound(const rap_plan* P, const Chain& ch, int64_t B, const int64_t* nnz) {
  int64_t b;
  if (ch.src_kind == SRC_SPARSE) {
    b = sat_add(nnz ? std::max<int64_t>(nnz[ch.src], 0) : 0, ch.has_fill ? B : 0);
  } else if (ch.src_kind == SRC_DENSE_BUCKET) {
    b = B;
  } else {
    const NGramDesc& ng = P->ngrams[ch.src];
    b = 0;
    for (int k = 0; k < ng.k; ++k) b = sat_add(b, chain_bound(P, P->chains[ng.chain[k]], B, nnz));
  }
  return std::min(b, sat_mul(ch.xcap, B));
}

double expected_len(const rap_plan* P, const Chain& ch, int64_t B, const int64_t* nnz) {
  double e;
  if (ch.src_kind == SRC_SPARSE) {
    // mean list length; a filled null row counts as one id (R10), so a
    // filled feature averages at least one id per row
    e = nnz && B > 0 ? (double)std::max<int64_t>(nnz[ch.src], 0) / (double)B : 1.0;
    if (ch.has_fill) e = std::max(e, 1.0);
  } else if (ch.src_kind == SRC_DENSE_BUCKET) {
    e = 1.0;
  } else {
    const NGramDesc& ng = P->ngrams[ch.src];
    e = 0;
    for (int k = 0; k < ng.k; ++k) e += expected_len(P, P->chains[ng.chain[k]], B, nnz);
  }
  return std::min(e, (double)ch.xcap);
}

int64_t values_bound(const rap_plan* P, int64_t B, const int64_t* nnz) {
  int64_t tot = 0;
  for (const SparseOut& so : P->souts) tot = sat_add(tot, chain_bound(P, P->chains[so.chain], B, nnz));
  return tot;
}

rap_status set_grid_budget(rap_plan* P, int32_t budget) {
  if (budget < 0 || budget > P->sm_count) return fail(RAP_ERR_INVALID_ARGUMENT, "sm_budget not in [0, #SMs]");
  P->budget = budget == 0 ? P->sm_count : budget;
  return RAP_OK;
}

// Bytes one call moves (each raw byte read once, each output byte written once).
double algorithmic_bytes(const rap_plan* P, int64_t B, const int64_t* nnz) {
  double b = 0;
  for (int c : P->used_dense) b += 4.0 * B + B / 8.0;
  for (int s : P->used_sparse) b += 4.0 * (B + 1) + 8.0 * (nnz ? nnz[s] : 0) + B / 8.0;
  b += 4.0 * B * P->d_out + 12.0 * B * P->souts.size() + 8.0 + 8.0 * values_bound(P, B, nnz);
  return b;
}

// ----------------------------------------------------------------------------
// Flattened device programs (rap_internal.h).

// Canonical form of a chain's id ops (rap_internal.h); ok = 0 when the ops
// are not an ordered subset of Clamp -> MapId -> SigridHash -> Bucketize.
// post = true: the chain is an NGram output (its ops follow the hash).
Canon make_canon(const DevOp* ops, const Chain& ch, int64_t tab_off, bool post) {
  Canon c;
  memset(&c, 0, sizeof(c));
  if (!post && ch.src_kind != SRC_SPARSE) return c;
  int stage = 0;
  for (int o = ch.op_begin; o < ch.op_end; ++o) {
    const DevOp& op = ops[o];
    int s, bit;
    switch (op.kind) {
      case OK_CLAMP: s = 0; bit = CB_CLAMP; c.lo = op.a; c.hi = op.b; break;
      case OK_MAPID:
        if (op.M) return Canon{};  // INT64_MIN key: interpreter
        s = 1; bit = CB_MAPID; c.map_a = op.a; c.map_m = op.m; c.map_def = op.b; break;
      case OK_SIGRID: s = 2; bit = CB_SIGRID; c.hs = op.hsalt; c.M = op.M; break;
      case OK_BUCKET_I: s = 3; bit = CB_BUCKET; c.bk_a = op.a; c.bk_m = op.m; break;
      case OK_BUCKET_S: s = 3; bit = CB_BUCKET; c.bk_a = tab_off + op.a; c.bk_m = op.m; break;
      default: return Canon{};
    }
    if (s < stage) return Canon{};
    stage = s + 1;
    c.mask |= bit;
    if (o >= ch.null_op_begin) c.null_mask |= bit;
  }
  c.ok = 1;
  return c;
}

// SProg of an id chain: the chain (and an NGram's source chains) with their
// ops copied in and rebased; the first Bucketize border tables that fit are
// staged next to the program.  Programs with more than kMaxStagedOps ops keep
// global op indices.
SProg make_sprog(rap_plan* P, int chain_idx) {
  SProg sp;
  memset(&sp, 0, sizeof(sp));
  sp.ch = P->chains[chain_idx];
  int nsrc = 0;
  if (sp.ch.src_kind == SRC_NGRAM) {
    sp.ng = P->ngrams[sp.ch.src];
    nsrc = sp.ng.k;
    for (int k = 0; k < nsrc; ++k) sp.src[k] = P->chains[sp.ng.chain[k]];
  }
  int total = 0;
  for (int c = 0; c <= nsrc; ++c) {
    const Chain& cc = c == 0 ? sp.ch : sp.src[c - 1];
    total += cc.op_end - cc.op_begin;
    if (cc.src_kind == SRC_DENSE_BUCKET) total += cc.dop_end - cc.dop_begin;
  }
  if (total > kMaxStagedOps) {
    sp.global_ops = 1;
    return sp;
  }
  int pos = 0;
  for (int c = 0; c <= nsrc; ++c) {
    Chain& cc = c == 0 ? sp.ch : sp.src[c - 1];
    if (cc.src_kind == SRC_DENSE_BUCKET) {
      const int n = cc.dop_end - cc.dop_begin;
      for (int k = 0; k < n; ++k) sp.ops[pos + k] = P->ops[cc.dop_begin + k];
      cc.dop_begin = pos;
      cc.dop_end = pos + n;
      pos += n;
    }
    const int n = cc.op_end - cc.op_begin;
    for (int k = 0; k < n; ++k) sp.ops[pos + k] = P->ops[cc.op_begin + k];
    cc.null_op_begin = pos + (cc.null_op_begin - cc.op_begin);
    cc.op_begin = pos;
    cc.op_end = pos + n;
    pos += n;
  }
  sp.n_ops = pos;
  std::vector<int64_t> tab;
  for (int o = 0; o < pos; ++o) {
    DevOp& op = sp.ops[o];
    if (op.kind == OK_BUCKET_I && (int)tab.size() + op.m <= kStageTab) {
      const int64_t local = (int64_t)tab.size();
      tab.insert(tab.end(), P->itab.begin() + op.a, P->itab.begin() + op.a + op.m);
      op.kind = OK_BUCKET_S;
      op.a = local;
    }
  }
  if (!tab.empty()) {
    if (P->itab.size() % 2) P->itab.push_back(0);  // 16-byte aligned for the staging copy
    sp.tab_off = (int64_t)P->itab.size();
    sp.tab_len = (int32_t)tab.size();
    P->itab.insert(P->itab.end(), tab.begin(), tab.end());
  }
  const DevOp* ops = sp.global_ops ? P->ops.data() : sp.ops;
  sp.cn = make_canon(ops, sp.ch, sp.tab_off, sp.ch.src_kind == SRC_NGRAM);
  for (int k = 0; k < nsrc; ++k) sp.src_cn[k] = make_canon(ops, sp.src[k], sp.tab_off, false);
  return sp;
}

// DProgs: dense outputs packed left to right into column groups of at most
// kGroupCols columns, kMaxDenseOps ops and kDenseTabF borders (a OneHot may
// be split across groups).
void build_dprogs(rap_plan* P, const std::vector<Unit>& flat) {
  std::vector<int> oprog_of(P->chains.size(), -1);
  DProg cur;
  memset(&cur, 0, sizeof(cur));
  auto close = [&](int end_col) {
    if (cur.n_units == 0) return;
    cur.width = end_col - cur.col0;
    P->dprogs.push_back(cur);
    memset(&cur, 0, sizeof(cur));
  };
  for (const Unit& u : flat) {
    // what one piece of this unit needs inside a DProg
    int need_ops = 0, need_tab = 0, kind = U_DENSE;
    const DenseExpr* de = nullptr;
    const Chain* ch = nullptr;
    if (u.kind == HU_DENSE) {
      de = &P->dexprs[u.idx];
      need_ops = de->op_end - de->op_begin;
    } else {
      ch = &P->chains[u.idx];
      if (ch->src_kind == SRC_DENSE_BUCKET) {
        kind = U_ONEHOT_DB;
        need_ops = (ch->dop_end - ch->dop_begin) + (ch->op_end - ch->op_begin);
        need_tab = ch->bm;
      } else {
        kind = U_ONEHOT_G;
        if (oprog_of[u.idx] < 0) {
          oprog_of[u.idx] = (int)P->oprogs.size();
          P->oprogs.push_back(make_sprog(P, u.idx));
        }
      }
    }
    const bool global = need_ops > kMaxDenseOps || need_tab > kDenseTabF;
    if (global) need_ops = need_tab = 0;
    int c = u.col, remaining = u.width;
    int64_t k0 = 0;
    while (remaining > 0) {
      if (cur.n_units == 0) cur.col0 = c;
      if (c - cur.col0 >= kGroupCols || cur.n_units == kGroupCols || cur.n_ops + need_ops > kMaxDenseOps ||
          cur.n_ftab + need_tab > kDenseTabF) {
        close(c);
        cur.col0 = c;
      }
      const int w = std::min(kGroupCols - (c - cur.col0), remaining);
      DUnit du;
      memset(&du, 0, sizeof(du));
      du.kind = kind;
      du.col = c - cur.col0;
      du.width = w;
      du.k0 = k0;
      du.gops = global ? 1 : 0;
      auto copy_ops = [&](int b, int e, int32_t* ob, int32_t* oe) {
        if (global) {
          *ob = b;
          *oe = e;
          return;
        }
        *ob = cur.n_ops;
        for (int k = b; k < e; ++k) cur.ops[cur.n_ops++] = P->ops[k];
        *oe = cur.n_ops;
      };
      auto slot_of = [&](int col) {
        for (int k = 0; k < cur.n_cols; ++k)
          if (cur.cols[k] == col) return k;
        cur.cols[cur.n_cols] = col;
        return cur.n_cols++;
      };
      if (kind == U_DENSE) {
        du.src_col = de->col;
        du.slot = slot_of(de->col);
        copy_ops(de->op_begin, de->op_end, &du.op_begin, &du.op_end);
      } else if (kind == U_ONEHOT_DB) {
        du.src_col = ch->src;
        du.slot = slot_of(ch->src);
        du.xcap = ch->xcap;
        copy_ops(ch->dop_begin, ch->dop_end, &du.op_begin, &du.op_end);
        copy_ops(ch->op_begin, ch->op_end, &du.iop_begin, &du.iop_end);
        du.bm = ch->bm;
        if (global) {
          du.btab = ch->btab;
        } else {
          du.btab = cur.n_ftab;
          for (int k = 0; k < ch->bm; ++k) cur.ftab[cur.n_ftab++] = P->ftab[ch->btab + k];
        }
      } else {
        du.prog = oprog_of[u.idx];
        du.xcap = ch->xcap;
      }
      cur.units[cur.n_units++] = du;
      if (kind != U_DENSE) cur.any_onehot = 1;
      c += w;
      k0 += w;
      remaining -= w;
    }
  }
  close(P->d_out);
}

// ----------------------------------------------------------------------------
// Row-block kernel descriptors (rap_internal.h RbFeat): closed-form length
// programs, emission kind, processing order and memo slots.

int clip32(int64_t x) { return (int)std::min<int64_t>(std::max<int64_t>(x, 0), INT32_MAX); }

// Canonical stage bits up to and including the highest bit of m (stage order
// Clamp -> MapId -> SigridHash -> Bucketize).
int stage_prefix(int m) {
  if (m == 0) return 0;
  int h = 0;
  for (int b = 0; b < 4; ++b)
    if (m & (1 << b)) h = b;
  return (2 << h) - 1;
}

bool same_stage_params(const rap_plan* P, const Canon& a, const Canon& b, int mask) {
  if ((mask & CB_CLAMP) && (a.lo != b.lo || a.hi != b.hi)) return false;
  if (mask & CB_MAPID) {
    if (a.map_m != b.map_m || a.map_def != b.map_def) return false;
    if (a.map_a != b.map_a &&
        memcmp(&P->itab[a.map_a], &P->itab[b.map_a], sizeof(int64_t) * 2 * ((size_t)1 << a.map_m)) != 0)
      return false;
  }
  if ((mask & CB_SIGRID) && (a.hs != b.hs || a.M != b.M)) return false;
  if (mask & CB_BUCKET) {
    if (a.bk_m != b.bk_m) return false;
    if (a.bk_a != b.bk_a && memcmp(&P->itab[a.bk_a], &P->itab[b.bk_a], sizeof(int64_t) * a.bk_m) != 0) return false;
  }
  return true;
}

// Does canonical list output O compute, as a prefix of its stages, the
// elements of NGram source chain S (same column, null rule and stage
// parameters)?  Returns the prefix mask, or -1.
int memo_prefix(const rap_plan* P, const Chain& o, const Canon& qo, const Chain& s, const Canon& qs) {
  if (o.src_kind != SRC_SPARSE || s.src_kind != SRC_SPARSE || o.src != s.src || !qo.ok || !qs.ok) return -1;
  if (o.has_fill != s.has_fill || (s.has_fill && o.fill != s.fill)) return -1;
  const int pm = stage_prefix(qs.mask);
  if ((qo.mask & pm) != qs.mask || (qo.null_mask & pm) != qs.null_mask) return -1;
  if (!same_stage_params(P, qs, qo, qs.mask)) return -1;
  return pm;
}

// The generated kernel's shared memory before id staging: the dense warp's
// 32-row tile after the base-phase totals (rap_jit.cpp tile_offset), no
// length cache, no shared memo.
// Warp-pair mode of the generated kernel (rap_rows_skel.cuh kPairs): two
// threads per row, each evaluating half of the outputs.
static int jit_pairs(const rap_plan* P) {
  static const int knob = [] {  // "0" / "1": force off / on (experiment knob; read once per process)
    const char* env = getenv("RAP_JIT_PAIRS");
    return env ? (env[0] == '1' ? 1 : 0) : 0;
  }();
  return knob && P->souts.size() >= 2 ? 1 : 0;
}
static int64_t jit_min_rows() {
  static const int64_t v = [] {  // (experiment knob; read once per process)
    const char* env = getenv("RAP_JIT_SMALL_B");
    return env ? (int64_t)atoll(env) : (int64_t)1 << 62;
  }();
  return v;
}
static int jit_pitch(const rap_plan*) { return 0; }
static int jit_threads(const rap_plan* P) {
  if (jit_pairs(P)) return 2 * kRbChunk;
  int r0 = 0;
  const int nd = jit_dense_warps(
      jit_dense_mode((int)P->souts.size(), P->d_out, (int)P->dprogs.size(), P->rb_dense_bytes, 0, &r0));
  return nd ? 224 + 32 * nd : kRbChunk;  // the generated kernel's CTA (rap_jit.cpp Gen::threads)
}
static int jit_base_smem(const rap_plan* P, int dense_bytes) {
  return rows_smem_bytes(dense_bytes, P->jit_max_fl, P->rb_max_cols, 0, (int)P->souts.size(), 0, 0, jit_pitch(P), 0,
                         P->jit_tab_bytes);
}
static int jit_tile_bytes(const rap_plan* P) {
  int r0 = 0;
  jit_dense_mode((int)P->souts.size(), P->d_out, (int)P->dprogs.size(), P->rb_dense_bytes, jit_pairs(P), &r0);
  return r0;
}
// Staged columns whose chunk ids the generated kernel bulk-copies into shared
// memory: as many as fit beside its base layout with two CTAs per SM.
static int jit_id_slots(const rap_plan* P) {
  // measured on C2 (B200): staging the ids cost 2.3 us of staging and gained
  // nothing in the emit phase (cold 59.5 vs 55.8 us), so it is opt-in
  const char* env = getenv("RAP_JIT_IDS");  // "1": stage the chunk ids (experiment knob)
  if (!(env && env[0] == '1')) return 0;
  const int budget = 113 * 1024 - jit_base_smem(P, std::max(P->jit_dense_bytes, jit_tile_bytes(P)));
  const int per = kRbIdCap * 8 + 8;
  return std::max(0, std::min(P->rb_max_cols, (budget - 16) / per));
}

JitPlanView jit_view(const rap_plan* P) {
  JitPlanView v;
  v.n_sparse_out = (int)P->souts.size();
  v.n_sparse_in = P->n_sparse_in;
  v.feat = P->rbfeat.data();
  v.sprogs = P->sprogs.data();
  v.perm = P->rb_perm.data();
  v.used_sparse = P->used_sparse.data();
  v.n_used_sparse = (int)P->used_sparse.size();
  v.dprogs = P->dprogs.data();
  v.n_dprogs = (int)P->dprogs.size();
  v.d_out = P->d_out;
  v.dense_bytes = P->rb_dense_bytes;
  v.itab = P->itab.data();
  v.ops = P->ops.data();
  v.ftab = P->ftab.data();
  v.id_slots = jit_id_slots(P);
  v.pairs = jit_pairs(P);
  return v;
}

constexpr int kRbMemoMax = 16;  // memo slots (256 rows x 8 bytes each) a CTA may hold

void build_rows(rap_plan* P) {
  const int F = (int)P->souts.size();
  P->rbfeat.assign(F, RbFeat{});
  std::vector<std::vector<int>> prov_out(F, std::vector<int>(kMaxNgramK, -1));
  for (int f = 0; f < F; ++f) {
    const Chain& ch = P->chains[P->souts[f].chain];
    const SProg& sp = P->sprogs[f];
    RbFeat& R = P->rbfeat[f];
    memset(&R, 0, sizeof(R));
    R.memo_slot = -1;
    for (int i = 0; i < kMaxNgramK; ++i) R.prov[i] = R.pslot[i] = -1;
    auto source = [&](int i, const Chain& c) {
      if (c.src_kind == SRC_SPARSE) {
        R.src[i] = c.src;
        R.cap[i] = clip32(c.xcap);
        R.ncap[i] = c.has_fill ? (int)std::min<int64_t>(1, c.null_xcap) : 0;
      } else {  // dense Bucketize source: one id (R4)
        R.src[i] = -1;
        R.cap[i] = (int)std::min<int64_t>(1, c.xcap);
      }
    };
    if (ch.src_kind == SRC_SPARSE) {
      R.kind = 0;
      R.k = 1;
      source(0, ch);
      R.emit = sp.cn.ok ? 0 : 1;
    } else if (ch.src_kind == SRC_DENSE_BUCKET) {
      R.kind = 1;
      R.out_cap = (int)std::min<int64_t>(1, ch.xcap);
      R.emit = 2;
    } else {
      const NGramDesc& ng = P->ngrams[ch.src];
      R.kind = 2;
      R.emit = 3;
      R.n = ng.n;
      R.k = ng.k;
      R.out_cap = clip32(ch.xcap);
      for (int i = 0; i < ng.k; ++i) source(i, P->chains[ng.chain[i]]);
    }
  }
  // memo providers: the first canonical list output whose stage prefix is the source chain
  std::vector<int> memo_mask(F, -1);
  for (int g = 0; g < F; ++g) {
    if (P->rbfeat[g].emit != 3) continue;
    const SProg& sp = P->sprogs[g];
    for (int k = 0; k < sp.ng.k; ++k) {
      const Chain& sc = P->chains[sp.ng.chain[k]];
      for (int f = 0; f < F; ++f) {
        if (P->rbfeat[f].emit != 0) continue;
        const int pm = memo_prefix(P, P->chains[P->souts[f].chain], P->sprogs[f].cn, sc, sp.src_cn[k]);
        if (pm < 0 || (memo_mask[f] >= 0 && memo_mask[f] != pm)) continue;
        memo_mask[f] = pm;
        prov_out[g][k] = f;
        break;
      }
    }
  }
  // processing order: an NGram right after the last of its providers
  struct Key {
    int a, b, c;
  };
  std::vector<Key> key(F);
  for (int f = 0; f < F; ++f) {
    int mp = -1;
    for (int k = 0; k < kMaxNgramK; ++k) mp = std::max(mp, prov_out[f][k]);
    key[f] = mp >= 0 ? Key{mp, 1, f} : Key{f, 0, f};
  }
  P->rb_perm.resize(F);
  std::iota(P->rb_perm.begin(), P->rb_perm.end(), 0);
  std::stable_sort(P->rb_perm.begin(), P->rb_perm.end(), [&](int x, int y) {
    if (key[x].a != key[y].a) return key[x].a < key[y].a;
    if (key[x].b != key[y].b) return key[x].b < key[y].b;
    return key[x].c < key[y].c;
  });
  std::vector<int> pidx(F);
  for (int i = 0; i < F; ++i) pidx[P->rb_perm[i]] = i;
  // memo slots: live from the provider to its last consumer (processing order)
  std::vector<int> last_use(F, -1);
  for (int g = 0; g < F; ++g)
    for (int k = 0; k < kMaxNgramK; ++k)
      if (prov_out[g][k] >= 0) last_use[prov_out[g][k]] = std::max(last_use[prov_out[g][k]], pidx[g]);
  std::vector<int> slot_of(F, -1), slot_end(kRbMemoMax, -1);
  int n_memo = 0;
  for (int i = 0; i < F; ++i) {
    const int f = P->rb_perm[i];
    if (last_use[f] < 0) continue;
    int sl = -1;
    for (int j = 0; j < kRbMemoMax && sl < 0; ++j)
      if (slot_end[j] < i) sl = j;
    if (sl < 0) continue;  // no free slot: the consumers recompute
    slot_end[sl] = last_use[f];
    slot_of[f] = sl;
    n_memo = std::max(n_memo, sl + 1);
    P->rbfeat[f].memo_slot = sl;
    P->rbfeat[f].memo_mask = memo_mask[f];
  }
  for (int g = 0; g < F; ++g)
    for (int k = 0; k < kMaxNgramK; ++k) {
      const int f = prov_out[g][k];
      if (f >= 0 && slot_of[f] >= 0) {
        P->rbfeat[g].prov[k] = pidx[f];
        P->rbfeat[g].pslot[k] = slot_of[f];
      }
    }
  P->rb_n_memo = n_memo;
  P->rb_all_cols = 0;
  for (int f = 0; f < F; ++f) {
    const RbFeat& R = P->rbfeat[f];
    const int kk = R.kind == 1 ? 0 : R.k;
    for (int i = 0; i < kk; ++i)
      if (R.src[i] >= 0 && R.src[i] < 64) P->rb_all_cols |= 1ull << R.src[i];
  }
  P->rb_fits = P->n_sparse_in <= kRbMaxCols && P->n_dense_in <= kRbMaxDense && F <= kRbMaxF;
  P->rb_max_fl = std::max(1, std::min(F, kRbMaxFL));
  P->jit_max_fl = std::max(1, std::min(F, kJitMaxF));
  P->rb_max_cols = std::max(1, (int)P->used_sparse.size());
}

}  // namespace

// ============================================================================
extern "C" {

const char* rap_status_string(rap_status s) {
  switch (s) {
    case RAP_OK: return "RAP_OK";
    case RAP_ERR_INVALID_ARGUMENT: return "RAP_ERR_INVALID_ARGUMENT";
    case RAP_ERR_INVALID_GRAPH: return "RAP_ERR_INVALID_GRAPH";
    case RAP_ERR_INVALID_PARAM: return "RAP_ERR_INVALID_PARAM";
    case RAP_ERR_CAPACITY: return "RAP_ERR_CAPACITY";
    case RAP_ERR_UNSUPPORTED: return "RAP_ERR_UNSUPPORTED";
    case RAP_ERR_CUDA: return "RAP_ERR_CUDA";
    case RAP_ERR_OUT_OF_MEMORY: return "RAP_ERR_OUT_OF_MEMORY";
  }
  return "RAP_ERR_UNKNOWN";
}

const char* rap_last_error(void) { return g_last_error.c_str(); }

// Host half of rap_plan_create (no device calls): lower every output of a
// validated graph to its device programs and row-block descriptors.
static rap_status plan_lower(const rap_graph* graph, const rap_op_param* params, const Validated& v, rap_plan* P) {
  rap_status st = RAP_OK;
  // ---- lower outputs
  Lowerer L{graph, params, P};
  L.dense_memo.assign(graph->n_nodes, -1);
  L.chain_memo.assign(graph->n_nodes, -1);
  L.type_of = v.type;
  int col = 0;
  std::vector<Unit> flat_units;
  for (int o = 0; o < graph->n_outputs; ++o) {
    const int node = graph->output_nodes[o];
    const int t = v.type[node];
    if (t == VT_DENSE) {
      Unit u{};
      u.kind = HU_DENSE;
      u.idx = L.lower_dense(node);
      u.col = col;
      u.width = 1;
      flat_units.push_back(u);
      col += 1;
    } else if (t == VT_VEC) {
      const rap_node& nd = graph->nodes[node];
      int c = L.lower_ids(nd.inputs[0], true, &st);
      if (c < 0) {
        return st;
      }
      Unit u{};
      u.kind = HU_ONEHOT;
      u.idx = c;
      u.col = col;
      u.width = params[nd.param].k_width;
      flat_units.push_back(u);
      col += u.width;
    } else {
      int c = L.lower_ids(node, true, &st);
      if (c < 0) {
        return st;
      }
      SparseOut so{};
      so.chain = c;
      so.rows_per_desc = kTileRows;
      P->souts.push_back(so);
    }
  }
  P->d_out = col;
  // ---- flattened device programs
  for (const SparseOut& so : P->souts) P->sprogs.push_back(make_sprog(P, so.chain));
  build_dprogs(P, flat_units);
  {
    int max_w = 1, max_cols = 1;
    for (const DProg& dp : P->dprogs) {
      max_w = std::max(max_w, dp.width);
      max_cols = std::max(max_cols, dp.n_cols);
    }
    const int rows = std::min(kDenseTileBytes / ((max_w | 1) * 4), kDenseInBytes / (max_cols * 4));
    P->rows_dense = std::max(32, std::min(256, rows / 32 * 32));
  }
  // raw columns the plan's outputs read (nodes reachable from them): the byte
  // model, and the columns a batch must supply (a sharded rank's plan reads
  // only its own tables' columns; the others may be NULL)
  {
    std::vector<char> ud(graph->n_dense_in, 0), us(graph->n_sparse_in, 0), seen(graph->n_nodes, 0);
    std::vector<int32_t> stack(graph->output_nodes, graph->output_nodes + graph->n_outputs);
    while (!stack.empty()) {
      const int32_t i = stack.back();
      stack.pop_back();
      if (i < 0 || i >= graph->n_nodes || seen[i]) continue;
      seen[i] = 1;
      for (int k = 0; k < graph->nodes[i].n_inputs; ++k) {
        int32_t r = graph->nodes[i].inputs[k];
        if (r < 0 && (-r) % 2 == 1) ud[(-r - 1) / 2] = 1;
        if (r < 0 && (-r) % 2 == 0) us[(-r - 2) / 2] = 1;
        if (r >= 0) stack.push_back(r);
      }
    }
    for (int c = 0; c < graph->n_dense_in; ++c)
      if (ud[c]) P->used_dense.push_back(c);
    for (int c = 0; c < graph->n_sparse_in; ++c)
      if (us[c]) P->used_sparse.push_back(c);
  }

  build_rows(P);
  return RAP_OK;
}

rap_status rap_plan_create(const rap_graph* graph, const rap_op_param* params, int32_t n_params, int32_t device,
                           int32_t sm_budget, rap_plan** out) {
  if (!out) return fail(RAP_ERR_INVALID_ARGUMENT, "out is NULL");
  *out = nullptr;
  Validated v;
  rap_status st = validate(graph, params, n_params, &v);
  if (st != RAP_OK) return st;
  if (graph->n_dense_in > 128 || graph->n_sparse_in > 1024)
    return fail(RAP_ERR_UNSUPPORTED, "more than 128 dense or 1024 sparse raw columns");

  int n_dev = 0;
  cudaError_t e = cudaGetDeviceCount(&n_dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceCount");
  if (device < 0 || device >= n_dev) return fail(RAP_ERR_INVALID_ARGUMENT, "bad device ordinal");
  DeviceGuard dg(device);

  rap_plan* P = new rap_plan();
  P->device = device;
  P->n_dense_in = graph->n_dense_in;
  P->n_sparse_in = graph->n_sparse_in;
  e = cudaDeviceGetAttribute(&P->sm_count, cudaDevAttrMultiProcessorCount, device);
  if (e != cudaSuccess) {
    delete P;
    return cuda_fail(e, "cudaDeviceGetAttribute");
  }
  st = set_grid_budget(P, sm_budget);
  if (st != RAP_OK) {
    delete P;
    return st;
  }

  st = plan_lower(graph, params, v, P);
  if (st != RAP_OK) {
    delete P;
    return st;
  }

  // ---- device blob
  std::vector<unsigned char> blob;
  P->off_ops = push_blob(blob, P->ops);
  P->off_sprogs = push_blob(blob, P->sprogs);
  P->off_oprogs = push_blob(blob, P->oprogs);
  P->off_dprogs = push_blob(blob, P->dprogs);
  P->off_ftab = push_blob(blob, P->ftab);
  P->off_itab = push_blob(blob, P->itab);
  P->off_rbfeat = push_blob(blob, P->rbfeat);
  P->off_perm = push_blob(blob, P->rb_perm);
  if (blob.empty()) blob.resize(16);
  e = cudaMalloc(&P->blob, blob.size());
  if (e == cudaSuccess) e = cudaMemcpy(P->blob, blob.data(), blob.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMalloc(&P->d_sched, 8 * sizeof(unsigned long long));
  if (e == cudaSuccess) {
    const unsigned long long init[8] = {0ull, 0ull, 0ull, 0ull, 0ull, 0ull, 0ull, 0ull};
    e = cudaMemcpy(P->d_sched, init, sizeof(init), cudaMemcpyHostToDevice);
  }
  if (e == cudaSuccess) e = cudaMalloc(&P->d_agg, kMaxCtas * sizeof(unsigned long long));
  if (e == cudaSuccess) e = cudaMemset(P->d_agg, 0, kMaxCtas * sizeof(unsigned long long));
  if (e == cudaSuccess) e = cudaMalloc(&P->d_part, kPartSlots * kPartLen * sizeof(int64_t));
  if (e == cudaSuccess) e = cudaMallocHost(&P->h_part, kPartSlots * kPartLen * sizeof(int64_t));
  if (e == cudaSuccess && P->rb_fits && !P->souts.empty()) {
    // agg [F][n_rb] + tot [F] + sup [F][kRbSupMax]
    const size_t n = (P->souts.size() + 1) * (size_t)kMaxCtas + P->souts.size() * (size_t)(1 + kRbSupMax);
    e = cudaMalloc(&P->d_agg_rb, n * sizeof(unsigned long long));
    if (e == cudaSuccess) e = cudaMemset(P->d_agg_rb, 0, n * sizeof(unsigned long long));
  }
  if (e == cudaSuccess) e = cudaMalloc(&P->d_err, sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMemset(P->d_err, 0, sizeof(int32_t));
  if (e != cudaSuccess) {
    rap_plan_destroy(P);
    return cuda_fail(e, "plan device allocation");
  }

  // ---- shared memory and occupancy
  int max_w = 1;
  for (const DProg& dp : P->dprogs) max_w = std::max(max_w, dp.width);
  P->smem = fused_smem_bytes(max_w);
  int occ = 0;
  e = (cudaError_t)fused_occupancy(P->smem, P->n_dense_in, P->n_sparse_in, &occ);
  if (e != cudaSuccess) {
    rap_plan_destroy(P);
    return cuda_fail(e, "occupancy query");
  }
  P->ctas_per_sm = std::max(1, occ);
  if (P->rb_fits) {
    P->rb_dense_bytes = rows_dense_bytes(max_w);
    P->rb_smem = rows_smem_bytes(P->rb_dense_bytes, P->rb_max_fl, P->rb_max_cols, P->rb_n_memo, (int)P->souts.size(), 1);
    // the generated kernel: no length cache, no shared memo (registers), and
    // only the dense tile when it generates the dense outputs (rap_jit.cpp)
    // the dense warp's 32-row tile after the base-phase totals (rap_jit.cpp tile_offset)
    P->jit_dense_bytes = jit_tile_bytes(P);
    P->jit_dense_bytes = std::max(P->jit_dense_bytes, jit_dense_need(jit_view(P)));  // + the emitter's memo rows
    P->jit_tab_bytes = jit_table_bytes(jit_view(P));
    P->jit_id_slots = jit_id_slots(P);
    P->jit_smem = rows_smem_bytes(P->jit_dense_bytes, P->jit_max_fl, P->rb_max_cols, 0, (int)P->souts.size(), 0,
                                  P->jit_id_slots, jit_pitch(P), 0, P->jit_tab_bytes);
    if (P->rb_smem > 227 * 1024) P->rb_fits = 0;
  }
  if (P->rb_fits) {
    int rocc = 0;
    e = (cudaError_t)rows_occupancy(P->rb_smem, &rocc);
    if (e != cudaSuccess) {
      rap_plan_destroy(P);
      return cuda_fail(e, "row-block kernel occupancy query");
    }
    P->rb_ctas_per_sm = rocc;
    if (rocc < 1) P->rb_fits = 0;  // shared memory does not fit one CTA
  }
  *out = P;
  return RAP_OK;
}

void rap_plan_destroy(rap_plan* P) {
  if (!P) return;
  DeviceGuard dg(P->device);
  cudaFree(P->blob);
  cudaFree(P->d_sched);
  cudaFree(P->d_agg);
  cudaFree(P->d_part);
  cudaFreeHost(P->h_part);
  cudaFree(P->d_err);
  cudaFree(P->d_trace);
  cudaFree(P->d_agg_rb);
  for (void* s : P->stage) cudaFree(s);
  delete P;
}

rap_status rap_set_budget(rap_plan* P, int32_t sm_budget) {
  if (!P) return fail(RAP_ERR_INVALID_ARGUMENT, "plan is NULL");
  return set_grid_budget(P, sm_budget);
}

rap_status rap_plan_output_shape(const rap_plan* P, int64_t n_rows, const int64_t* sp_nnz, int64_t* d_out_cols,
                                 int64_t* n_sparse_out, int64_t* values_upper_bound) {
  if (!P) return fail(RAP_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (n_rows < 0) return fail(RAP_ERR_INVALID_ARGUMENT, "n_rows < 0");
  if (!sp_nnz && n_rows > 0 && P->n_sparse_in > 0) return fail(RAP_ERR_INVALID_ARGUMENT, "sp_nnz is NULL");
  if (d_out_cols) *d_out_cols = P->d_out;
  if (n_sparse_out) *n_sparse_out = (int64_t)P->souts.size();
  if (values_upper_bound) *values_upper_bound = n_rows > 0 ? values_bound(P, n_rows, sp_nnz) : 0;
  return RAP_OK;
}

rap_status rap_debug_trace(rap_plan* P, int32_t enable, uint64_t* host_out, int64_t cap, int64_t* n_desc) {
  if (!P) return fail(RAP_ERR_INVALID_ARGUMENT, "plan is NULL");
  DeviceGuard dg(P->device);
  cudaError_t e = cudaSuccess;
  if (enable == 1) {
    if (cap <= 0) return fail(RAP_ERR_INVALID_ARGUMENT, "cap <= 0");
    e = cudaDeviceSynchronize();
    if (e == cudaSuccess && P->trace_cap < cap) {
      cudaFree(P->d_trace);
      P->d_trace = nullptr;
      P->trace_cap = 0;
      e = cudaMalloc(&P->d_trace, sizeof(unsigned long long) * kTracePts * cap);
      if (e == cudaSuccess) P->trace_cap = cap;
    }
    if (e == cudaSuccess) e = cudaMemset(P->d_trace, 0, sizeof(unsigned long long) * kTracePts * P->trace_cap);
  } else if (enable == 0) {
    if (!host_out) return fail(RAP_ERR_INVALID_ARGUMENT, "host_out is NULL");
    e = cudaDeviceSynchronize();
    const int64_t n = std::min(cap, std::min(P->trace_cap, P->last_n_desc));
    if (e == cudaSuccess && n > 0)
      e = cudaMemcpy(host_out, P->d_trace, sizeof(unsigned long long) * kTracePts * n, cudaMemcpyDeviceToHost);
    if (n_desc) *n_desc = P->last_n_desc;
  } else {
    e = cudaDeviceSynchronize();
    cudaFree(P->d_trace);
    P->d_trace = nullptr;
    P->trace_cap = 0;
  }
  return e == cudaSuccess ? RAP_OK : cuda_fail(e, "rap_debug_trace");
}

rap_status rap_plan_info_get(const rap_plan* P, rap_plan_info* info) {
  if (!P || !info) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  memset(info, 0, sizeof(*info));
  info->device = P->device;
  info->sm_count = P->sm_count;
  info->sm_budget = P->budget;
  info->ctas_per_sm = P->ctas_per_sm;
  info->threads_per_cta = kThreads;
  info->grid = P->budget * P->ctas_per_sm;
  info->n_dense_out_cols = P->d_out;
  info->n_sparse_out = (int32_t)P->souts.size();
  info->n_dense_groups = (int32_t)P->dprogs.size();
  info->rows_per_dense_desc = kDenseBlockRows;
  int rmax = 0, rmin = INT32_MAX;
  for (const SparseOut& so : P->souts) {
    rmax = std::max(rmax, so.rows_per_desc);
    rmin = std::min(rmin, so.rows_per_desc);
  }
  info->max_rows_per_sparse_desc = rmax;
  info->min_rows_per_sparse_desc = P->souts.empty() ? 0 : rmin;
  info->n_descriptors_last = P->last_n_desc;
  info->n_launches = P->n_launches;
  info->smem_bytes = P->smem;
  info->kernel_mode = P->kernel_mode;
  info->kernel_last = P->kernel_last;
  info->rows_ctas_per_sm = P->rb_fits ? P->rb_ctas_per_sm : 0;
  info->rows_smem_bytes = P->rb_smem;
  info->rb_row_blocks = P->rb_last_n_rb;
  info->rb_feature_groups = P->rb_last_n_fg;
  info->rb_rows = P->rb_last_rows;
  info->rb_memo_slots = P->rb_n_memo;
  info->partition_uploads = P->partition_uploads;
  info->jit_state = P->jit_state;
  info->jit_ctas_per_sm = P->jit_ctas_per_sm;
  info->jit_compile_seconds = P->jit_s;
  if (P->kernel_last == RAP_KERNEL_ROWS || P->kernel_last == RAP_KERNEL_JIT) info->grid = P->rb_last_grid;
  return RAP_OK;
}

rap_status rap_set_kernel(rap_plan* P, int32_t mode) {
  if (!P) return fail(RAP_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (mode != RAP_KERNEL_AUTO && mode != RAP_KERNEL_TILED && mode != RAP_KERNEL_ROWS && mode != RAP_KERNEL_JIT)
    return fail(RAP_ERR_INVALID_ARGUMENT, "unknown kernel mode");
  if ((mode == RAP_KERNEL_ROWS || mode == RAP_KERNEL_JIT) && !P->rb_fits && !P->souts.empty())
    return fail(RAP_ERR_UNSUPPORTED, "plan does not fit the row-block kernel (> 64 sparse / 32 dense raw columns)");
  P->kernel_mode = mode;
  return RAP_OK;
}

rap_status rap_debug_jit_source(const rap_graph* graph, const rap_op_param* params, int32_t n_params, char* buf,
                                int64_t cap, int32_t compile, int32_t* ok) {
  if (ok) *ok = 0;
  Validated v;
  rap_status st = validate(graph, params, n_params, &v);
  if (st != RAP_OK) return st;
  rap_plan* P = new rap_plan();
  P->n_dense_in = graph->n_dense_in;
  P->n_sparse_in = graph->n_sparse_in;
  st = plan_lower(graph, params, v, P);
  if (st == RAP_OK) {
    int max_w = 1;
    for (const DProg& dp : P->dprogs) max_w = std::max(max_w, dp.width);
    P->rb_dense_bytes = rows_dense_bytes(max_w);
  }
  if (st == RAP_OK && (!P->rb_fits || P->souts.empty()))
    st = fail(RAP_ERR_UNSUPPORTED, "plan does not fit the row-block kernel");
  if (st == RAP_OK) {
    const std::string src = jit_generate(jit_view(P));
    if (buf && cap > 0) {
      const size_t n = std::min<size_t>(src.size(), (size_t)cap - 1);
      memcpy(buf, src.data(), n);
      buf[n] = 0;
    }
    if (compile) {
      std::string log;
      const bool good = jit_compile_only(src, &log);
      if (ok) *ok = good ? 1 : 0;
      g_last_error = log;
    }
  }
  delete P;
  return st;
}

rap_status rap_check_overflow(rap_plan* P, int32_t* overflow) {
  if (!P || !overflow) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  DeviceGuard dg(P->device);
  cudaError_t e = cudaDeviceSynchronize();
  int32_t v = 0;
  if (e == cudaSuccess) e = cudaMemcpy(&v, P->d_err, sizeof(v), cudaMemcpyDeviceToHost);
  if (e == cudaSuccess) e = cudaMemset(P->d_err, 0, sizeof(int32_t));
  if (e != cudaSuccess) return cuda_fail(e, "rap_check_overflow");
  *overflow = v ? 1 : 0;
  return RAP_OK;
}

static rap_status check_batch(const rap_plan* P, const rap_raw_batch* raw, const rap_output* out) {
  if (!P || !raw || !out) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  if (out->flags & ~(RAP_OUT_CHAIN | RAP_OUT_VALUES_I32)) return fail(RAP_ERR_INVALID_ARGUMENT, "unknown output flags");
  if ((out->flags & RAP_OUT_CHAIN) && (out->flags & RAP_OUT_VALUES_I32))
    return fail(RAP_ERR_UNSUPPORTED, "RAP_OUT_VALUES_I32 with RAP_OUT_CHAIN");
  if (raw->n_rows < 0) return fail(RAP_ERR_INVALID_ARGUMENT, "n_rows < 0");
  if (raw->n_rows > (int64_t)INT32_MAX - kTileRows) return fail(RAP_ERR_INVALID_ARGUMENT, "n_rows too large");
  const int64_t B = raw->n_rows;
  if (B == 0) {
    if (!P->souts.empty() && !out->offsets) return fail(RAP_ERR_INVALID_ARGUMENT, "offsets NULL");
    return RAP_OK;
  }
  for (int c : P->used_dense)
    if (!raw->dense || !raw->dense[c]) return fail(RAP_ERR_INVALID_ARGUMENT, "dense column pointer NULL");
  for (int s : P->used_sparse)
    if (!raw->sp_offsets || !raw->sp_values || !raw->sp_offsets[s])
      return fail(RAP_ERR_INVALID_ARGUMENT, "sparse column pointer NULL");
  if (P->d_out > 0 && (!out->dense_out || out->dense_ld < P->d_out))
    return fail(RAP_ERR_INVALID_ARGUMENT, "dense_out NULL or dense_ld < d_out");
  if (!P->souts.empty()) {
    if (!out->lengths || !out->offsets) return fail(RAP_ERR_INVALID_ARGUMENT, "lengths/offsets NULL");
    if (P->n_sparse_in > 0 && !raw->sp_nnz) return fail(RAP_ERR_INVALID_ARGUMENT, "sp_nnz NULL");
    const int64_t bound = values_bound(P, B, raw->sp_nnz);
    if (bound > 0 && !out->values) return fail(RAP_ERR_INVALID_ARGUMENT, "values NULL");
    if (out->values_capacity < bound)
      return fail(RAP_ERR_CAPACITY, "values_capacity " + std::to_string(out->values_capacity) + " < bound " +
                                        std::to_string(bound));
  }
  return RAP_OK;
}

// ----------------------------------------------------------------------------
// Cost model of the fused kernel (lane-instructions per row).
// It plays the role of the paper's preprocessing latency predictor
// (L1037-1057) for the intra-kernel schedule: the partition gives every CTA
// about the same predicted work.
// Units: ~0.03 ns of one CTA slot per row; calibrated on B200 against the
// per-feature phase times of scripts/trace.py (C2 graph: a Clamp+SigridHash
// row ~2.8 ns, +MapId ~5.6 ns, +Bucketize(1024) ~5.3 ns, a trigram ~15.6 ns).
static double op_cost(const DevOp& op) {
  switch (op.kind) {
    case OK_CLAMP: return 8;
    case OK_SIGRID: return 40;
    case OK_MAPID: return 126;
    case OK_BUCKET_I:
    case OK_BUCKET_S: return 4 + 8 * std::log2((double)op.m + 1);
    case OK_FILL_F: return 3;
    case OK_LOGIT: return 40;
    default: return 70;  // OK_BOXCOX
  }
}

static double chain_ops_cost(const rap_plan* P, const Chain& ch) {
  double c = 0;
  for (int o = ch.op_begin; o < ch.op_end; ++o) c += op_cost(P->ops[o]);
  if (ch.src_kind == SRC_DENSE_BUCKET) {
    for (int o = ch.dop_begin; o < ch.dop_end; ++o) c += op_cost(P->ops[o]);
    c += 4 + 6 * std::log2((double)ch.bm + 1);
  }
  return c;
}

static double sparse_row_cost(const rap_plan* P, const Chain& ch, int64_t B, const int64_t* nnz) {
  if (ch.src_kind != SRC_NGRAM) return 40 + expected_len(P, ch, B, nnz) * (8 + chain_ops_cost(P, ch));
  const NGramDesc& ng = P->ngrams[ch.src];
  double c = 40, lens = 0, elem = 0;
  for (int k = 0; k < ng.k; ++k) {
    const Chain& s = P->chains[ng.chain[k]];
    const double e = expected_len(P, s, B, nnz);
    lens += e;
    elem += e * (8 + chain_ops_cost(P, s));
    c += 15;
  }
  const double windows = std::min((double)ch.xcap, std::max(0.0, lens - ng.n + 1));
  return c + windows * (ng.n * (elem / std::max(lens, 1.0) + 90) + 10 + chain_ops_cost(P, ch));
}

static double dense_row_cost(const rap_plan* P, const DProg& dp) {
  double c = 0;
  for (int u = 0; u < dp.n_units; ++u) {
    const DUnit& un = dp.units[u];
    const DevOp* ops = un.gops ? P->ops.data() : dp.ops;
    c += 12;
    if (un.kind == U_ONEHOT_G) {
      c += 100;
      continue;
    }
    for (int o = un.op_begin; o < un.op_end; ++o) c += op_cost(ops[o]);
    if (un.kind == U_ONEHOT_DB) {
      c += 10 + 6 * std::log2((double)un.bm + 1);
      for (int o = un.iop_begin; o < un.iop_end; ++o) c += op_cost(ops[o]);
    }
  }
  return c + 2.0 * dp.width;
}

// Split the sparse tile sequence (feature-major, the scan order) into `grid`
// contiguous ranges of about equal predicted cost.  The key is
// (rows, grid, each used source's mean list length quantised to 2^(1/4)
// steps), so batches of the same shape reuse the uploaded table.
static rap_status update_partition(rap_plan* P, int64_t B, const int64_t* nnz, int64_t S, int64_t D, int grid,
                                   cudaStream_t stream, const int64_t** d_part_out) {
  std::vector<int64_t> key = {B, grid};
  (void)D;
  // a launch captured into a CUDA graph bakes in its slot (and, on a miss, the
  // upload from the pinned staging slot): such slots are pinned for the plan's
  // lifetime, so later eager calls never overwrite what a replay reads
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(stream, &cap) != cudaSuccess) {
    cudaGetLastError();
    cap = cudaStreamCaptureStatusNone;
  }
  const bool capturing = cap != cudaStreamCaptureStatusNone;
  auto use = [&](size_t i) {
    if (capturing) P->part_pin[i] = 1;
    *d_part_out = P->d_part + i * kPartLen;
    return RAP_OK;
  };
  for (int s : P->used_sparse) {
    const double m = nnz && B > 0 ? (double)std::max<int64_t>(nnz[s], 0) / (double)B : 0.0;
    key.push_back(m <= 1.0 / 64 ? -1000 : (int64_t)std::lround(4.0 * std::log2(m)));
  }
  for (size_t i = 0; i < P->part_keys.size(); ++i)
    if (P->part_keys[i] == key) return use(i);
  // A partition only balances work: any cached one with the same rows and grid
  // covers exactly the same tiles, so a batch whose quantised mean lengths are
  // within one step of a cached shape reuses it (no re-plan, upload or slot
  // eviction when a mean sits on a quantisation boundary and flips from batch
  // to batch).
  for (size_t i = 0; i < P->part_keys.size(); ++i) {
    const std::vector<int64_t>& k = P->part_keys[i];
    if (k.size() != key.size() || k[0] != key[0] || k[1] != key[1]) continue;
    bool near = true;
    for (size_t j = 2; j < k.size() && near; ++j) near = std::llabs(k[j] - key[j]) <= 1;
    if (near) return use(i);
  }
  const int64_t F = (int64_t)P->souts.size();
  const int64_t T = F ? S / F : 0;
  const double kTileFixed = 400.0;  // per-unit overhead (lane-instructions)
  std::vector<double> fcost(F);
  for (int64_t f = 0; f < F; ++f) fcost[f] = sparse_row_cost(P, P->chains[P->souts[f].chain], B, nnz);
  auto unit_cost = [&](int64_t u) -> double {
    const int64_t f = u / T, rt = u - f * T;
    const int64_t rows = std::min<int64_t>(kTileRows, B - rt * kTileRows);
    return kTileFixed + (double)rows * fcost[f];
  };
  const int64_t U = S;
  double W = 0;
  for (int64_t u = 0; u < U; ++u) W += unit_cost(u);
  // One contiguous cost-balanced range per WARP (grid x kWarps slots; a CTA
  // owns the ranges of its 8 warps): warps of a CTA finish together, so no
  // warp idles at the CTA's barriers.  Dense blocks go round robin over the
  // ranks (block d to rank d mod grid) and are not charged here: the CTAs of
  // an SM share its issue slots, so a dense block mostly fills slots its SM
  // neighbours leave idle (measured: charging it made C2 slower).
  int slot = -1;
  const bool evict = (int)P->part_keys.size() == kPartSlots;
  if (!evict) {
    slot = (int)P->part_keys.size();
  } else {
    for (int k = 0; k < kPartSlots && slot < 0; ++k) {
      const int c = (P->part_next + k) % kPartSlots;
      if (!P->part_pin[c]) slot = c;
    }
    if (slot < 0) return fail(RAP_ERR_UNSUPPORTED, "every partition slot is pinned by a captured CUDA graph");
    // an eviction syncs the stream (the staging slot may feed an in-flight
    // upload), which a capture cannot do
    if (capturing) return fail(RAP_ERR_UNSUPPORTED, "a new batch shape during CUDA-graph capture needs a free "
                                                   "partition slot: launch each shape once before capturing");
  }
  P->part_next = (slot + 1) % kPartSlots;
  int64_t* part = P->h_part + (size_t)slot * kPartLen;
  const int n = grid * kWarpsPerCta;
  // evicting: the pinned slot may still feed an in-flight upload (only
  // after kPartSlots distinct batch shapes; never in steady state)
  cudaError_t e = cudaSuccess;
  if (evict) e = cudaStreamSynchronize(stream);
  if (e != cudaSuccess) return cuda_fail(e, "partition slot reuse");
  part[0] = 0;
  double acc = 0;
  int64_t u = 0;
  for (int c = 1; c < n; ++c) {
    const double target = W * (double)c / (double)n;
    while (u < U && acc + 0.5 * unit_cost(u) < target) acc += unit_cost(u++);
    part[c] = u;
  }
  part[n] = U;
  int64_t* d = P->d_part + (size_t)slot * kPartLen;
  e = cudaMemcpyAsync(d, part, sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, stream);
  if (e != cudaSuccess) return cuda_fail(e, "partition upload");
  P->partition_uploads += 1;
  if ((int)P->part_keys.size() < kPartSlots) {
    P->part_keys.push_back(key);
    P->part_pin.push_back(0);
  } else {
    P->part_keys[slot] = key;
  }
  if (capturing) P->part_pin[slot] = 1;
  *d_part_out = d;
  return RAP_OK;
}

// The generated kernel of this plan (rap_jit.cpp), variant `small`: built on
// first use; on failure the plan keeps the interpreted row-block kernel.
static bool jit_ready(rap_plan* P, int i) {  // i: variant (bit 0 small, bit 1 int32 values)
  if (P->jit_st[i] == 0) {
    const char* env = getenv("RAP_JIT");
    if (env && env[0] == '0') {
      P->jit_st[i] = -1;
    } else {
      char log[2048] = {0};
      JitModule* m = jit_build(jit_view(P), i, log, (int)sizeof(log));
      int occ = 0;
      if (m && jit_occupancy(m, P->jit_smem, jit_threads(P), &occ) == 0 && occ >= 1) {
        P->jit[i] = m;
        P->jit_occ[i] = occ;
        P->jit_s += jit_compile_seconds(m);
        P->jit_st[i] = 1;
      } else {
        P->jit_st[i] = -1;
        g_last_error = std::string("generated kernel unavailable: ") + log;
      }
    }
  }
  P->jit_state = P->jit_st[i];
  P->jit_ctas_per_sm = P->jit_occ[i];
  return P->jit_st[i] == 1;
}

// Does this batch go to the row-block kernel?  RAP_KERNEL_AUTO: when the plan
// fits it and every used raw sparse column averages <= 2 ids per row (the
// row-per-thread mapping is efficient for short lists; long multi-hot lists
// go element-parallel through the tiled kernel).
static bool use_rows(const rap_plan* P, int64_t B, const int64_t* nnz) {
  if (P->kernel_mode == RAP_KERNEL_TILED || !P->rb_fits || P->souts.empty()) return false;
  if (P->kernel_mode == RAP_KERNEL_ROWS || P->kernel_mode == RAP_KERNEL_JIT) return true;
  for (int s : P->used_sparse)
    if (nnz && B > 0 && (double)nnz[s] > 2.0 * (double)B) return false;
  return true;
}

// Row-block geometry of one launch (rap_internal.h RbGeom): row blocks of a
// multiple of 32 rows and feature groups (contiguous ranges of the processing
// order, balanced by the cost model, <= kRbMaxFL outputs each), at most the
// budget's CTA slots.  Large batches: one feature group, one row block per
// slot.  Small batches: 256-row blocks, the slots left over split the outputs.
// n_dense_tiles > 0 (the interpreted form): when the dense blocks are few
// (<= a quarter of the slots) each gets a dedicated CTA, so small batches run
// the dense outputs beside the sparse phases rather than after them.
static void rows_geometry(const rap_plan* P, int64_t B, const int64_t* nnz, int ctas_per_sm, RbGeom* g,
                          int64_t n_dense_tiles = 0, int budget = 0, bool one_group = false) {
  const int F = (int)P->souts.size();
  const int bud = budget > 0 ? budget : P->budget;
  int64_t slots = std::max<int64_t>(1, std::min<int64_t>((int64_t)bud * ctas_per_sm, kMaxCtas));
  g->n_dcta = 0;
  g->id_slots = 0;
  if (n_dense_tiles > 0 && n_dense_tiles <= slots / 4) {
    g->n_dcta = (int)n_dense_tiles;
    slots -= n_dense_tiles;
  }
  const int fg_min = (F + kRbMaxFL - 1) / kRbMaxFL;
  const int64_t nb256 = (B + kRbChunk - 1) / kRbChunk;
  int64_t n_rb, n_fg;
  if (one_group || nb256 * fg_min * 2 >= slots) {  // one_group: the generated kernel (one group of every output)
    n_fg = one_group ? 1 : fg_min;
    n_rb = std::max<int64_t>(1, std::min<int64_t>(slots / n_fg, (B + 31) / 32));
  } else {
    n_rb = nb256;
    n_fg = std::max<int64_t>(fg_min, std::min<int64_t>({(int64_t)F, (int64_t)kRbMaxFg, slots / n_rb}));
  }
  static const int64_t knob_rows = [] {  // experiment knob: rows per block (read once per process)
    const char* env = getenv("RAP_RB_ROWS");
    return env ? std::max<int64_t>(32, atoll(env) / 32 * 32) : (int64_t)0;
  }();
  int64_t rows = knob_rows ? knob_rows : 32 * ((B + 32 * n_rb - 1) / (32 * n_rb));
  n_rb = std::max<int64_t>(1, (B + rows - 1) / rows);
  if (n_rb * n_fg > kMaxCtas) {  // knob out of range: back to the default
    rows = 32 * ((B + 32 * (kMaxCtas / n_fg) - 1) / (32 * (kMaxCtas / n_fg)));
    n_rb = (B + rows - 1) / rows;
  }
  g->n_rb = (int)n_rb;
  g->rows_rb = (int)rows;
  // feature groups: contiguous ranges of the processing order, equal predicted cost
  std::vector<double> cost(F);
  double W = 0;
  for (int i = 0; i < F; ++i) {
    cost[i] = sparse_row_cost(P, P->chains[P->souts[P->rb_perm[i]].chain], B, nnz);
    W += cost[i];
  }
  int gcount = 0, start = 0;
  double acc = 0;
  g->fg_off[0] = 0;
  for (int i = 0; i < F; ++i) {
    const bool full = !one_group && i - start >= kRbMaxFL;
    const bool due = gcount + 1 < n_fg && acc + 0.5 * cost[i] >= W * (double)(gcount + 1) / (double)n_fg && i > start;
    if ((full || due) && gcount + 1 < kRbMaxFg) {
      g->fg_off[++gcount] = i;
      start = i;
    }
    acc += cost[i];
  }
  g->fg_off[++gcount] = F;
  g->n_fg = gcount;
}

static rap_status launch(rap_plan* P, const rap_raw_batch* raw, const rap_output* out, cudaStream_t stream) {
  const int64_t B = raw->n_rows;
  cudaError_t e;
  if (B == 0) {
    if (out->offsets && !(out->flags & RAP_OUT_CHAIN)) {  // offsets[F * 0] = 0, also when F = 0
      e = cudaMemsetAsync(out->offsets, 0, sizeof(int64_t), stream);
      if (e != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync");
    }
    return RAP_OK;
  }
  // Work decomposition: 128-row sparse tiles per output, then
  // 128-row dense blocks per column group; one contiguous cost-balanced unit
  // range per CTA.
  const int64_t F = (int64_t)P->souts.size();
  const int64_t T = (B + kTileRows - 1) / kTileRows;
  const int64_t n_sparse_tiles = F * T;
  int64_t drow0 = 0, drows = B;
  rap_shard_rows(B, P->rank, P->world, &drow0, &drows);
  const int64_t n_dense = P->dprogs.empty() ? 0 : (int64_t)P->dprogs.size() * ((drows + kDenseBlockRows - 1) / kDenseBlockRows);
  if (n_sparse_tiles == 0 && n_dense == 0) {
    // nothing to compute (a rank without tables or rows): offsets = [0] (R17)
    if (out->offsets && !(out->flags & RAP_OUT_CHAIN)) {
      e = cudaMemsetAsync(out->offsets, 0, sizeof(int64_t), stream);
      if (e != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync");
    }
    return RAP_OK;
  }
  Common c{};
  c.ops = reinterpret_cast<const DevOp*>(P->blob + P->off_ops);
  c.sprogs = reinterpret_cast<const SProg*>(P->blob + P->off_sprogs);
  c.oprogs = reinterpret_cast<const SProg*>(P->blob + P->off_oprogs);
  c.dprogs = reinterpret_cast<const DProg*>(P->blob + P->off_dprogs);
  c.ftab = reinterpret_cast<const float*>(P->blob + P->off_ftab);
  c.itab = reinterpret_cast<const int64_t*>(P->blob + P->off_itab);
  c.n_sparse_out = (int32_t)F;
  c.n_groups = (int32_t)P->dprogs.size();
  c.n_rows = B;
  c.tiles_per_feature = T;
  c.n_sparse_tiles = n_sparse_tiles;
  c.n_dense_tiles = n_dense;
  c.dense_row0 = drow0;
  c.n_dense_rows = drows;
  c.chain = (out->flags & RAP_OUT_CHAIN) ? 1 : 0;
  c.vi32 = (out->flags & RAP_OUT_VALUES_I32) ? 1 : 0;
  c.sched = P->d_sched;
  c.agg = P->d_agg;
  c.dense_out = out->dense_out;
  c.ld = out->dense_ld;
  c.lengths = out->lengths;
  c.offsets = out->offsets;
  c.values = out->values;
  c.values_cap = out->values_capacity;
  c.err = P->d_err;
  c.trace = P->d_trace;
  c.trace_cap = P->trace_cap;
  LaunchRaw lr{};
  lr.n_dense = P->n_dense_in;
  lr.n_sparse = P->n_sparse_in;
  lr.dense = raw->dense;
  lr.dvalid = raw->dense_valid;
  lr.off = raw->sp_offsets;
  lr.val = raw->sp_values;
  lr.svalid = raw->sp_valid;
  if (use_rows(P, B, raw->sp_nnz)) {
    RbGeom g;
    memset(&g, 0, sizeof(g));
    // 32-bit scans when every offset of this launch fits 31 bits
    const bool small = !c.chain && values_bound(P, B, raw->sp_nnz) < (int64_t)INT32_MAX - 1;
    const bool want_jit = P->kernel_mode == RAP_KERNEL_JIT || P->kernel_mode == RAP_KERNEL_AUTO;
    const int iv = (small ? 1 : 0) | (c.vi32 ? 2 : 0);
    const bool jit = want_jit && jit_ready(P, iv);
    // the generated kernel: one group of every output over as many row blocks
    // as the budget's slots hold (RAP_JIT_SMALL_B: below this batch size the
    // interpreted form's feature groups fill the slots instead)
    // (more outputs than an interpreted group holds: the generated kernel's one
    // group takes up to kJitMaxF of them)
    const int Fp = (int)P->souts.size();
    const bool jit_geo = jit && (Fp > kRbMaxFL ? Fp <= kJitMaxF : (B >= jit_min_rows() || jit_pairs(P)));
    rows_geometry(P, B, raw->sp_nnz, jit ? P->jit_occ[iv] : P->rb_ctas_per_sm, &g, 0, 0, jit_geo);
    if (!jit || !(g.n_fg == 1 && drow0 == 0 && drows == B))  // interpreted form: its geometry, dense CTAs
      rows_geometry(P, B, raw->sp_nnz, P->rb_ctas_per_sm, &g, n_dense);
    g.max_fl = P->rb_max_fl;
    g.max_cols = P->rb_max_cols;
    g.dense_bytes = P->rb_dense_bytes;
    g.n_memo = P->rb_n_memo;
    g.small = small ? 1 : 0;
    g.all_cols = P->rb_all_cols;
    g.feat = reinterpret_cast<const RbFeat*>(P->blob + P->off_rbfeat);
    g.perm = reinterpret_cast<const int32_t*>(P->blob + P->off_perm);
    g.agg = P->d_agg_rb;
    g.tot = P->d_agg_rb + (P->souts.size() + 1) * (size_t)kMaxCtas;
    g.sup = g.tot + P->souts.size();
    g.sched = P->d_sched + 4;
    // the generated policy covers one group of every output, over the batch's
    // own rows (a sharded plan's dense shard runs the interpreted form)
    const bool gen = jit && g.n_fg == 1 && drow0 == 0 && drows == B;
    if (gen) {
      g.n_dcta = 0;  // the generated form evaluates the dense outputs itself
      g.len_cache = 0;
      g.n_memo = 0;
      g.dense_bytes = P->jit_dense_bytes;
      g.max_fl = P->jit_max_fl;
      g.id_slots = P->jit_id_slots;
      g.pitch = jit_pitch(P);
      g.feat_recs = 0;
    } else {
      g.len_cache = 1;
      g.pitch = 0;
      g.feat_recs = 1;
    }
    int rc = gen ? launch_jit(P->jit[iv], c, g, lr, P->jit_smem, jit_threads(P), stream)
                 : launch_rows(c, g, lr, P->rb_smem, stream);
    if (rc != 0) return cuda_fail((cudaError_t)rc, gen ? "generated kernel launch" : "row-block kernel launch");
    P->kernel_last = gen ? RAP_KERNEL_JIT : RAP_KERNEL_ROWS;
    P->rb_last_n_rb = g.n_rb;
    P->rb_last_n_fg = g.n_fg;
    P->rb_last_grid = g.n_rb * g.n_fg + g.n_dcta;
    P->rb_last_rows = g.rows_rb;
    P->n_launches += 1;
    P->last_n_desc = (int64_t)g.n_rb * g.n_fg;
    return RAP_OK;
  }
  // tiled kernel: grid = the budget's CTA slots, but no more CTAs than there
  // is work for (a warp per sparse tile, a CTA per dense block): small
  // batches then pay a shorter aggregate chain and fewer idle CTAs
  const int64_t want = std::max<int64_t>(1, std::max<int64_t>(n_dense, (n_sparse_tiles + kWarpsPerCta - 1) / kWarpsPerCta));
  const int64_t grid = std::min<int64_t>(std::min<int64_t>((int64_t)P->budget * P->ctas_per_sm, kMaxCtas), want);
  const int64_t* d_part = nullptr;
  rap_status pst = update_partition(P, B, raw->sp_nnz, n_sparse_tiles, n_dense, (int)grid, stream, &d_part);
  if (pst != RAP_OK) return pst;
  c.part = d_part;
  const int64_t n_total = n_sparse_tiles + n_dense;
  int rc = launch_fused(c, lr, (int)grid, P->smem, stream);
  if (rc != 0) return cuda_fail((cudaError_t)rc, "fused kernel launch");
  P->kernel_last = RAP_KERNEL_TILED;
  P->n_launches += 1;
  P->last_n_desc = n_total;
  return RAP_OK;
}

rap_status rap_preprocess(rap_plan* P, const rap_raw_batch* raw, const rap_output* out, void* stream) {
  rap_status st = check_batch(P, raw, out);
  if (st != RAP_OK) return st;
  DeviceGuard dg(P->device);
  return launch(P, raw, out, reinterpret_cast<cudaStream_t>(stream));
}

static rap_status stage_buf(rap_plan* P, size_t slot, size_t bytes, void** ptr) {
  if (P->stage.size() <= slot) {
    P->stage.resize(slot + 1, nullptr);
    P->stage_cap.resize(slot + 1, 0);
  }
  if (P->stage_cap[slot] < bytes) {
    cudaFree(P->stage[slot]);
    P->stage[slot] = nullptr;
    size_t cap = std::max<size_t>(bytes + bytes / 4, 256);
    cudaError_t e = cudaMalloc(&P->stage[slot], cap);
    if (e != cudaSuccess) {
      P->stage_cap[slot] = 0;
      return fail(RAP_ERR_OUT_OF_MEMORY, "staging allocation");
    }
    P->stage_cap[slot] = cap;
  }
  *ptr = P->stage[slot];
  return RAP_OK;
}

static rap_status preprocess_host_impl(rap_plan* P, const rap_raw_batch* raw, const rap_output* out, void* stream_v,
                                       bool sync) {
  rap_status st = check_batch(P, raw, out);
  if (st != RAP_OK) return st;
  DeviceGuard dg(P->device);
  cudaStream_t stream = reinterpret_cast<cudaStream_t>(stream_v);
  const int64_t B = raw->n_rows;
  const size_t bm_bytes = (size_t)((B + 31) / 32) * 4;
  std::vector<const float*> d_dense(P->n_dense_in, nullptr);
  std::vector<const uint32_t*> d_dvalid(P->n_dense_in, nullptr);
  std::vector<const int32_t*> d_off(P->n_sparse_in, nullptr);
  std::vector<const int64_t*> d_val(P->n_sparse_in, nullptr);
  std::vector<const uint32_t*> d_svalid(P->n_sparse_in, nullptr);
  size_t slot = 0;
  cudaError_t e = cudaSuccess;
  // the columns' H2D copies are collected, then issued as one gather launch
  // when every source is device-mapped pinned memory (launch_gather_h2d), else
  // one cudaMemcpyAsync each
  std::vector<const void*> c_src;
  std::vector<void*> c_dst;
  std::vector<int64_t> c_bytes;
  auto h2d = [&](const void* src, size_t bytes, void** dst) -> rap_status {
    rap_status s = stage_buf(P, slot++, bytes, dst);
    if (s != RAP_OK) return s;
    if (bytes) {
      c_src.push_back(src);
      c_dst.push_back(*dst);
      c_bytes.push_back((int64_t)bytes);
    }
    return RAP_OK;
  };
  if (B > 0) {
    for (int c : P->used_dense) {
      void* d;
      if ((st = h2d(raw->dense[c], sizeof(float) * B, &d)) != RAP_OK) return st;
      d_dense[c] = static_cast<const float*>(d);
      if (raw->dense_valid && raw->dense_valid[c]) {
        if ((st = h2d(raw->dense_valid[c], bm_bytes, &d)) != RAP_OK) return st;
        d_dvalid[c] = static_cast<const uint32_t*>(d);
      }
    }
    for (int s : P->used_sparse) {
      void* d;
      const int32_t* ho = raw->sp_offsets[s];
      if ((st = h2d(ho, sizeof(int32_t) * (B + 1), &d)) != RAP_OK) return st;
      d_off[s] = static_cast<const int32_t*>(d);
      const int64_t lo = ho[0], n = ho[B] - ho[0];
      if ((st = h2d(raw->sp_values[s] + lo, sizeof(int64_t) * std::max<int64_t>(n, 0), &d)) != RAP_OK) return st;
      d_val[s] = static_cast<const int64_t*>(d) - lo;  // absolute offsets index this base
      if (raw->sp_valid && raw->sp_valid[s]) {
        if ((st = h2d(raw->sp_valid[s], bm_bytes, &d)) != RAP_OK) return st;
        d_svalid[s] = static_cast<const uint32_t*>(d);
      }
    }
  }
  if (!c_src.empty()) {
    static const bool copies = [] {  // "1": one cudaMemcpyAsync per column (experiment knob; read once per process)
      const char* env = getenv("RAP_H2D_COPIES");
      return env && env[0] == '1';
    }();
    std::vector<const void*> mapped(c_src.size(), nullptr);
    bool all_mapped = !copies;
    for (size_t i = 0; all_mapped && i < c_src.size(); ++i) {
      cudaPointerAttributes pa;
      all_mapped = cudaPointerGetAttributes(&pa, c_src[i]) == cudaSuccess && pa.type == cudaMemoryTypeHost &&
                   pa.devicePointer != nullptr;
      if (all_mapped) mapped[i] = pa.devicePointer;
    }
    cudaGetLastError();  // pageable pointers leave a sticky-free error behind
    if (all_mapped) {
      e = (cudaError_t)launch_gather_h2d(mapped.data(), c_dst.data(), c_bytes.data(), (int)c_src.size(), stream);
      if (e != cudaSuccess) return cuda_fail(e, "H2D gather");
    } else {
      for (size_t i = 0; i < c_src.size(); ++i) {
        e = cudaMemcpyAsync(c_dst[i], c_src[i], (size_t)c_bytes[i], cudaMemcpyHostToDevice, stream);
        if (e != cudaSuccess) return cuda_fail(e, "H2D copy");
      }
    }
  }
  const int64_t F = (int64_t)P->souts.size();
  // the staging values buffer is sized from the ids the host offsets hold
  // (not the caller's sp_nnz, which may understate them)
  std::vector<int64_t> host_nnz(std::max(P->n_sparse_in, 1), 0);
  for (int s = 0; s < P->n_sparse_in; ++s)
    if (raw->sp_offsets && raw->sp_offsets[s] && B > 0)
      host_nnz[s] = std::max<int64_t>(raw->sp_nnz ? raw->sp_nnz[s] : 0,
                                      (int64_t)raw->sp_offsets[s][B] - (int64_t)raw->sp_offsets[s][0]);
  const int64_t vb = B > 0 ? values_bound(P, B, host_nnz.data()) : 0;
  int64_t drow0 = 0, drows = B;
  rap_shard_rows(B, P->rank, P->world, &drow0, &drows);
  void *dd = nullptr, *dl = nullptr, *dof = nullptr, *dv = nullptr;
  if ((st = stage_buf(P, slot++, sizeof(float) * std::max<int64_t>(drows * P->d_out, 1), &dd)) != RAP_OK) return st;
  if ((st = stage_buf(P, slot++, sizeof(int32_t) * std::max<int64_t>(B * F, 1), &dl)) != RAP_OK) return st;
  if ((st = stage_buf(P, slot++, sizeof(int64_t) * (B * F + 1), &dof)) != RAP_OK) return st;
  if ((st = stage_buf(P, slot++, sizeof(int64_t) * std::max<int64_t>(vb, 1), &dv)) != RAP_OK) return st;
  rap_raw_batch dr = *raw;
  dr.dense = d_dense.data();
  dr.dense_valid = d_dvalid.data();
  dr.sp_offsets = d_off.data();
  dr.sp_values = d_val.data();
  dr.sp_valid = d_svalid.data();
  rap_output dout{};
  dout.dense_out = static_cast<float*>(dd);
  dout.dense_ld = P->d_out;
  dout.lengths = static_cast<int32_t*>(dl);
  dout.offsets = static_cast<int64_t*>(dof);
  dout.values = static_cast<int64_t*>(dv);
  dout.values_capacity = std::max<int64_t>(vb, 0);
  if ((st = launch(P, &dr, &dout, stream)) != RAP_OK) return st;
  // D2H
  static const bool d2h_gather = [] {  // "1": fixed-size outputs by one SM copy launch into mapped host memory (experiment knob)
    const char* env = getenv("RAP_D2H_GATHER");
    return env && env[0] == '1';
  }();
  bool fixed_done = false;
  if (d2h_gather && out->dense_ld == P->d_out && !(out->flags & RAP_OUT_CHAIN)) {
    const void* src[3];
    void* dst[3];
    int64_t nb[3];
    int n = 0;
    bool ok = true;
    auto add = [&](const void* d, void* h, int64_t bytes) {
      if (bytes <= 0 || !ok) return;
      cudaPointerAttributes pa;
      if (h == nullptr || cudaPointerGetAttributes(&pa, h) != cudaSuccess || pa.type != cudaMemoryTypeHost ||
          pa.devicePointer == nullptr) {
        ok = false;
        return;
      }
      src[n] = d;
      dst[n] = pa.devicePointer;
      nb[n++] = bytes;
    };
    if (drows > 0 && P->d_out > 0) add(dd, out->dense_out, (int64_t)sizeof(float) * drows * P->d_out);
    if (F > 0 && B > 0) add(dl, out->lengths, (int64_t)sizeof(int32_t) * B * F);
    if (F > 0) add(dof, out->offsets, (int64_t)sizeof(int64_t) * (B * F + 1));
    cudaGetLastError();
    if (ok && n > 0) {
      e = (cudaError_t)launch_gather_h2d(src, dst, nb, n, stream);
      if (e != cudaSuccess) return cuda_fail(e, "D2H gather");
      fixed_done = true;
    }
  }
  if (!fixed_done && drows > 0 && P->d_out > 0) {
    if (out->dense_ld == P->d_out)
      e = cudaMemcpyAsync(out->dense_out, dd, sizeof(float) * drows * P->d_out, cudaMemcpyDeviceToHost, stream);
    else
      e = cudaMemcpy2DAsync(out->dense_out, sizeof(float) * out->dense_ld, dd, sizeof(float) * P->d_out,
                            sizeof(float) * P->d_out, drows, cudaMemcpyDeviceToHost, stream);
    if (e != cudaSuccess) return cuda_fail(e, "D2H dense");
  }
  if (F > 0) {
    if (B > 0 && !fixed_done)
      e = cudaMemcpyAsync(out->lengths, dl, sizeof(int32_t) * B * F, cudaMemcpyDeviceToHost, stream);
    if (e == cudaSuccess && !fixed_done)
      e = cudaMemcpyAsync(out->offsets, dof, sizeof(int64_t) * (B * F + 1), cudaMemcpyDeviceToHost, stream);
    if (e == cudaSuccess && vb > 0) {
      // exact count: pinned host memory is device-mapped (UVA), so a copy
      // kernel reads the total on the device and moves only the written ids;
      // pageable memory gets the bounded copy
      cudaPointerAttributes pa;
      const bool pinned = cudaPointerGetAttributes(&pa, out->values) == cudaSuccess && pa.type == cudaMemoryTypeHost &&
                          pa.devicePointer != nullptr && (reinterpret_cast<uintptr_t>(out->values) & 15) == 0;
      cudaGetLastError();
      if (pinned && !(out->flags & RAP_OUT_CHAIN)) {
        const int rc = launch_values_to_host(static_cast<const int64_t*>(dv), static_cast<const int64_t*>(dof) + B * F,
                                             std::min<int64_t>(vb, out->values_capacity),
                                             static_cast<int64_t*>(pa.devicePointer), stream);
        e = (cudaError_t)rc;
      } else {
        e = cudaMemcpyAsync(out->values, dv, sizeof(int64_t) * vb, cudaMemcpyDeviceToHost, stream);
      }
    }
    if (e != cudaSuccess) return cuda_fail(e, "D2H sparse");
  } else if (out->offsets) {
    out->offsets[0] = 0;  // no sparse outputs: the single total (HOST buffer)
  }
  if (!sync) return RAP_OK;
  e = cudaStreamSynchronize(stream);
  if (e != cudaSuccess) return cuda_fail(e, "cudaStreamSynchronize");
  return RAP_OK;
}

rap_status rap_preprocess_host(rap_plan* P, const rap_raw_batch* raw, const rap_output* out, void* stream) {
  if (out && (out->flags & RAP_OUT_VALUES_I32)) return fail(RAP_ERR_UNSUPPORTED, "RAP_OUT_VALUES_I32: rap_preprocess only");
  return preprocess_host_impl(P, raw, out, stream, true);
}

rap_status rap_preprocess_host_async(rap_plan* P, const rap_raw_batch* raw, const rap_output* out, void* stream) {
  if (out && (out->flags & RAP_OUT_VALUES_I32)) return fail(RAP_ERR_UNSUPPORTED, "RAP_OUT_VALUES_I32: rap_preprocess only");
  return preprocess_host_impl(P, raw, out, stream, false);
}

// ---- latency model (the paper's preprocessing latency predictor, §5.2
// L1037-1057, for one fused launch at an SM budget) ----
// The model replays the launch the plan would make (kernel, geometry) and
// charges a fixed part, the busiest CTA's predicted work and the bytes:
//   T(b) = t0[k] + c_work[k] * work(b) + c_pair[k] * pairs(b) + bytes / BW
// with work the CTA's cost units (the tiled kernel's partition model) and
// pairs its (sparse output, row) pairs (the row-block kernels: whole
// 224/256-row chunks).  Least-squares fits to B200 kernel times over budgets
// 8..148 for configs 1, 2 and 4 at several batch sizes (scripts/budget_sweep.py
// -> scripts/fit_cost_model.py, profiles/r02_cost_model_fit.txt): the tiled
// kernel is explained by work, the row-block kernels by pairs (a per-output
// latency, not the op mix).  RAP_MODEL="t0,c_work,c_pair x 3 kernels,bw_gbs"
// overrides the constants (refitting).
struct PredTerms {
  int family;      // RAP_KERNEL_TILED / _ROWS / _JIT
  int64_t grid;    // CTAs
  double work;     // sparse cost units of the busiest CTA
  double bytes;    // algorithmic bytes of the launch
  double dwork;    // dense cost units of that CTA (the generated kernel: its dense warp's)
  double pairs;    // (sparse output, row) pairs of that CTA: a per-output latency the cost units miss
};

static PredTerms predict_terms(const rap_plan* P, int64_t B, const int64_t* nnz, int b) {
  PredTerms t{RAP_KERNEL_TILED, 0, 0.0, B > 0 ? algorithmic_bytes(P, B, nnz) : 0.0, 0.0, 0.0};
  if (B <= 0) return t;
  const int F = (int)P->souts.size();
  std::vector<double> fc(F);
  double sparse = 0;
  for (int f = 0; f < F; ++f) sparse += (fc[f] = sparse_row_cost(P, P->chains[P->souts[f].chain], B, nnz));
  int64_t drow0 = 0, drows = B;
  rap_shard_rows(B, P->rank, P->world, &drow0, &drows);
  double dense = 0;
  for (const DProg& dp : P->dprogs) dense += dense_row_cost(P, dp);
  const int64_t n_dense = P->dprogs.empty() ? 0 : (int64_t)P->dprogs.size() * ((drows + kDenseBlockRows - 1) / kDenseBlockRows);
  if (use_rows(P, B, nnz)) {
    const bool small = values_bound(P, B, nnz) < (int64_t)INT32_MAX - 1;
    const int iv = small ? 1 : 0;
    const bool want_jit = (P->kernel_mode == RAP_KERNEL_JIT || P->kernel_mode == RAP_KERNEL_AUTO) && P->jit_st[iv] != -1;
    RbGeom g;
    memset(&g, 0, sizeof(g));
    const int jocc = P->jit_occ[iv] > 0 ? P->jit_occ[iv] : P->rb_ctas_per_sm;
    rows_geometry(P, B, nnz, want_jit ? jocc : P->rb_ctas_per_sm, &g, 0, b,
                  want_jit && F > kRbMaxFL && F <= kJitMaxF);  // as launch(): one group beyond kRbMaxFL
    const bool jit = want_jit && g.n_fg == 1 && drow0 == 0 && drows == B;
    if (!jit) rows_geometry(P, B, nnz, P->rb_ctas_per_sm, &g, n_dense, b);
    const int chunk = jit ? 224 : kRbChunk;
    const int64_t chunks = (g.rows_rb + chunk - 1) / chunk;
    double gmax = 0;  // the costliest feature group's cost per row
    int fmax = 0;
    for (int k = 0; k < g.n_fg; ++k) {
      double c = 0;
      for (int i = g.fg_off[k]; i < g.fg_off[k + 1]; ++i) c += fc[P->rb_perm[i]];
      if (c > gmax) {
        gmax = c;
        fmax = g.fg_off[k + 1] - g.fg_off[k];
      }
    }
    t.pairs = (double)fmax * (double)(chunks * chunk);
    if (jit && chunks == 1) {  // the dense-warp tail (rap_jit.cpp tail_split) takes ~20 % of the outputs' cost
      int r0 = 0;
      if (jit_dense_mode((int)P->souts.size(), P->d_out, (int)P->dprogs.size(), P->rb_dense_bytes, jit_pairs(P), &r0) == 3)
        t.pairs *= 0.8;
    }
    t.family = jit ? RAP_KERNEL_JIT : RAP_KERNEL_ROWS;
    t.grid = (int64_t)g.n_rb * g.n_fg + g.n_dcta;
    t.work = gmax * (double)(chunks * chunk);
    if (jit) {
      int r0 = 0;
      const int dm = jit_dense_mode((int)P->souts.size(), P->d_out, (int)P->dprogs.size(), P->rb_dense_bytes,
                                    jit_pairs(P), &r0);
      const int64_t rows = std::min<int64_t>(g.rows_rb, B);
      // mode 2: every warp one 32-row tile at a time (the busiest warp's rows,
      // before the grid wait); mode 1: the dense warp takes the block's rows
      // mode 3: the dense warps run beside the sparse phases (hidden: their
      // rows per warp stay well below the sparse warps' chain); mode 2 / 1:
      // the busiest warp's dense rows add to the launch
      const int nd = dm == 2 ? jit_dense_tiles(jit_pairs(P)) : std::max(1, jit_dense_warps(dm));
      t.dwork = dm == 3 ? 0.0 : dense * 32.0 * (double)((rows + 32 * nd - 1) / (32 * nd));
    } else if (g.n_dcta > 0) {
      t.dwork = dense * (double)kDenseBlockRows;  // one dense block per dedicated CTA
    } else if (n_dense > 0) {
      t.dwork = dense * (double)drows / (double)std::max<int64_t>(1, t.grid);  // round robin
    }
    return t;
  }
  const int64_t T = (B + kTileRows - 1) / kTileRows;
  const int64_t want = std::max<int64_t>(1, std::max<int64_t>(n_dense, ((int64_t)F * T + kWarpsPerCta - 1) / kWarpsPerCta));
  t.grid = std::min<int64_t>(std::min<int64_t>((int64_t)b * P->ctas_per_sm, kMaxCtas), want);
  t.work = sparse * (double)B / (double)t.grid;
  t.dwork = dense * (double)drows / (double)t.grid;
  t.pairs = (double)F * (double)B / (double)t.grid;
  return t;
}

constexpr int kModelK = 13;
static void model_constants(double k[kModelK]) {
  // per kernel (tiled, rows, generated): t0 (us), c_work (us per cost unit),
  // c_pair (us per (output, row) pair), c_dense (us per dense cost unit of
  // the busiest CTA's serial dense work); then the HBM bandwidth (GB/s)
  static const double fit[kModelK] = {RAP_MODEL_FIT};
  for (int i = 0; i < kModelK; ++i) k[i] = fit[i];
  if (const char* env = getenv("RAP_MODEL")) {
    double v[kModelK];
    if (sscanf(env, "%lf,%lf,%lf,%lf,%lf,%lf,%lf,%lf,%lf,%lf,%lf,%lf,%lf", &v[0], &v[1], &v[2], &v[3], &v[4], &v[5],
               &v[6], &v[7], &v[8], &v[9], &v[10], &v[11], &v[12]) == kModelK)
      for (int i = 0; i < kModelK; ++i) k[i] = v[i];
  }
}

rap_status rap_predict_terms(const rap_plan* P, int64_t n_rows, const int64_t* sp_nnz, int32_t sm_budget,
                             double* terms) {
  if (!P || !terms) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  if (n_rows < 0 || sm_budget < 0 || sm_budget > P->sm_count) return fail(RAP_ERR_INVALID_ARGUMENT, "bad size");
  if (n_rows > 0 && P->n_sparse_in > 0 && !sp_nnz) return fail(RAP_ERR_INVALID_ARGUMENT, "sp_nnz NULL");
  const PredTerms t = predict_terms(P, n_rows, sp_nnz, sm_budget == 0 ? P->sm_count : sm_budget);
  terms[0] = t.family;
  terms[1] = (double)t.grid;
  terms[2] = t.work;
  terms[3] = t.bytes;
  terms[4] = t.dwork;
  terms[5] = t.pairs;
  return RAP_OK;
}

rap_status rap_predict_latency_us(const rap_plan* P, int64_t n_rows, const int64_t* sp_nnz, int32_t sm_budget,
                                  double* latency_us) {
  if (!P || !latency_us) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  double terms[6];
  rap_status st = rap_predict_terms(P, n_rows, sp_nnz, sm_budget, terms);
  if (st != RAP_OK) return st;
  if (n_rows == 0) {
    *latency_us = 0.0;
    return RAP_OK;
  }
  double k[kModelK];
  model_constants(k);
  const int fam = (int)terms[0];
  const int i = fam == RAP_KERNEL_JIT ? 8 : fam == RAP_KERNEL_ROWS ? 4 : 0;
  *latency_us = k[i] + k[i + 1] * terms[2] + k[i + 2] * terms[5] + k[i + 3] * terms[4] + terms[3] / (k[12] * 1e3);
  return RAP_OK;
}

rap_status rap_choose_budget(const rap_plan* P, int64_t n_rows, const int64_t* sp_nnz, double oc_us,
                             int32_t* sm_budget, double* t_delta_us) {
  if (!P || !sm_budget) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  // T_delta = sum_i P_i - OC (L1138-1143); pick the smallest budget with
  // T_delta <= 0 so the most SMs stay with training (L1145-1152).
  double best_td = 1e300;
  int best_b = P->sm_count;
  for (int b = 1; b <= P->sm_count; ++b) {
    double p_us = 0;
    rap_status st = rap_predict_latency_us(P, n_rows, sp_nnz, b, &p_us);
    if (st != RAP_OK) return st;
    const double td = p_us - oc_us;
    if (td <= 0) {
      *sm_budget = b;
      if (t_delta_us) *t_delta_us = td;
      return RAP_OK;
    }
    if (td < best_td) {
      best_td = td;
      best_b = b;
    }
  }
  *sm_budget = best_b;
  if (t_delta_us) *t_delta_us = best_td;
  return RAP_OK;
}

}  // extern "C"

// ----------------------------------------------------------------------------
// Multi-GPU (§7.2, hybrid parallelism
// L488-499).

rap_status rap_shard_rows(int64_t n_rows, int32_t rank, int32_t world, int64_t* row0, int64_t* rows) {
  if (!row0 || !rows) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  if (n_rows < 0 || world < 1 || rank < 0 || rank >= world) return fail(RAP_ERR_INVALID_ARGUMENT, "bad shard");
  if (world == 1) {
    *row0 = 0;
    *rows = n_rows;
    return RAP_OK;
  }
  // boundary r = floor(n_rows * r / world) rounded down to 128 rows; the last
  // rank ends at n_rows
  auto bound = [&](int32_t r) -> int64_t {
    if (r >= world) return n_rows;
    const int64_t b = (int64_t)((__int128)n_rows * r / world);
    return b / kTileRows * kTileRows;
  };
  *row0 = bound(rank);
  *rows = bound(rank + 1) - *row0;
  return RAP_OK;
}

rap_status rap_plan_output_costs(const rap_plan* P, int64_t n_rows, const int64_t* sp_nnz, double* cost) {
  if (!P || !cost) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  if (n_rows < 0) return fail(RAP_ERR_INVALID_ARGUMENT, "n_rows < 0");
  for (size_t f = 0; f < P->souts.size(); ++f)
    cost[f] = (double)n_rows * sparse_row_cost(P, P->chains[P->souts[f].chain], n_rows, sp_nnz);
  return RAP_OK;
}

static rap_status place_impl(const double* cost, const int32_t* colocate, int32_t n, int32_t world, int32_t mode,
                             int64_t n_rows, double imbalance_tol, const rap_comm_model* comm, int32_t* owner_out,
                             double* load_out, rap_residual* residual);

rap_status rap_place(const double* cost, const int32_t* colocate, int32_t n, int32_t world, int32_t mode,
                     int64_t n_rows, double imbalance_tol, int32_t* owner_out, double* load_out,
                     rap_residual* residual) {
  return place_impl(cost, colocate, n, world, mode, n_rows, imbalance_tol, nullptr, owner_out, load_out, residual);
}

// Joint mapping (§7.2; include/rap.h).  A group = an
// output and the outputs colocated with it (an NGram with its first source's
// table) moves as one preprocessing graph.
rap_status rap_place_joint(const double* cost, const int32_t* colocate, const int32_t* home, int32_t n,
                           int32_t world, int64_t n_rows, const rap_comm_model* comm, double oc_us,
                           int32_t* owner_out, double* time_out, int32_t* n_moves) {
  if (n < 0 || world < 1 || n_rows < 0) return fail(RAP_ERR_INVALID_ARGUMENT, "bad size");
  if (n > 0 && (!cost || !home || !owner_out)) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  if (!comm || !(comm->us_per_unit > 0) || !(comm->link_gbs > 0) || !(comm->link_latency_us >= 0) ||
      (n > 0 && !comm->row_bytes))
    return fail(RAP_ERR_INVALID_ARGUMENT, "comm model: us_per_unit, link_gbs > 0, link_latency_us >= 0, row_bytes");
  std::vector<int> anchor(n);
  for (int j = 0; j < n; ++j) {
    if (!(cost[j] >= 0)) return fail(RAP_ERR_INVALID_ARGUMENT, "cost must be >= 0");
    if (home[j] < -1 || home[j] >= world) return fail(RAP_ERR_INVALID_ARGUMENT, "home[j] must be -1 or a rank");
    const int c = colocate ? colocate[j] : -1;
    if (c >= j || c < -1) return fail(RAP_ERR_INVALID_ARGUMENT, "colocate[j] must be -1 or < j");
    anchor[j] = c < 0 ? j : anchor[c];
    if (home[j] != home[anchor[j]]) return fail(RAP_ERR_INVALID_ARGUMENT, "colocated outputs must share their home");
  }
  // groups: cost (us), exchange time when away from home (us), home
  std::vector<int> gid(n, -1), ghome;
  std::vector<double> gus, gxus;
  for (int j = 0; j < n; ++j) {
    if (anchor[j] == j) {
      gid[j] = (int)ghome.size();
      ghome.push_back(home[j]);
      gus.push_back(0.0);
      gxus.push_back(comm->link_latency_us);
    }
    const int g = gid[anchor[j]];
    gid[j] = g;
    gus[g] += cost[j] * comm->us_per_unit;
    if (!(comm->row_bytes[j] >= 0)) return fail(RAP_ERR_INVALID_ARGUMENT, "row_bytes must be >= 0");
    gxus[g] += (double)n_rows * comm->row_bytes[j] / (1e3 * comm->link_gbs);
  }
  const int G = (int)ghome.size();
  std::vector<int> gown(ghome);  // the data-locality mapping (L1524-1529)
  // rank times: a duplicated graph (home -1, not moved) runs on every rank; a
  // moved graph costs its compute and its exchange on the rank that runs it
  auto times = [&](const std::vector<int>& own, std::vector<double>* T) {
    T->assign(world, 0.0);
    for (int g = 0; g < G; ++g) {
      if (own[g] < 0) {
        for (int r = 0; r < world; ++r) (*T)[r] += gus[g];
      } else {
        (*T)[own[g]] += gus[g] + (own[g] != ghome[g] ? gxus[g] : 0.0);
      }
    }
  };
  auto score = [&](const std::vector<double>& T) {  // (exposed, makespan)
    double e = 0, m = 0;
    for (double t : T) {
      e = std::max(e, std::max(0.0, t - oc_us));
      m = std::max(m, t);
    }
    return std::make_pair(e, m);
  };
  std::vector<double> T;
  times(gown, &T);
  auto best = score(T);
  int moves = 0;
  for (int it = 0; it < 4 * G + 4 && world > 1; ++it) {
    int h = 0, l = 0;
    for (int r = 0; r < world; ++r) {
      if (T[r] > T[h]) h = r;
      if (T[r] < T[l]) l = r;
    }
    if (h == l) break;
    // substitution: the graph on h whose move to l lowers the cost most
    int bg = -1;
    std::pair<double, double> bs = best;
    for (int g = 0; g < G; ++g) {
      if (gown[g] != h) continue;
      std::vector<int> own = gown;
      own[g] = l;
      std::vector<double> T2;
      times(own, &T2);
      const auto sc = score(T2);
      if (sc.first < bs.first - 1e-9 || (sc.first <= bs.first + 1e-9 && sc.second < bs.second - 1e-9)) {
        bs = sc;
        bg = g;
      }
    }
    if (bg < 0) break;  // no substitution improves the mapping (L1600-1602)
    gown[bg] = l;
    times(gown, &T);
    best = bs;
    ++moves;
  }
  for (int j = 0; j < n; ++j) owner_out[j] = gown[gid[j]];
  if (time_out)
    for (int r = 0; r < world; ++r) time_out[r] = T[r];
  if (n_moves) *n_moves = moves;
  return RAP_OK;
}

rap_status rap_place_comm(const double* cost, const int32_t* colocate, int32_t n, int32_t world, int32_t mode,
                          int64_t n_rows, const rap_comm_model* comm, int32_t* owner_out, double* load_out,
                          rap_residual* residual) {
  if (comm && (!(comm->us_per_unit > 0) || !(comm->link_gbs > 0) || !(comm->link_latency_us >= 0) ||
               (n > 0 && !comm->row_bytes)))
    return fail(RAP_ERR_INVALID_ARGUMENT, "comm model: us_per_unit, link_gbs > 0, link_latency_us >= 0, row_bytes");
  return place_impl(cost, colocate, n, world, mode, n_rows, 0.0, comm, owner_out, load_out, residual);
}

static rap_status place_impl(const double* cost, const int32_t* colocate, int32_t n, int32_t world, int32_t mode,
                             int64_t n_rows, double imbalance_tol, const rap_comm_model* comm, int32_t* owner_out,
                             double* load_out, rap_residual* residual) {
  if (n < 0 || world < 1 || n_rows < 0) return fail(RAP_ERR_INVALID_ARGUMENT, "bad size");
  if (n > 0 && (!cost || !owner_out)) return fail(RAP_ERR_INVALID_ARGUMENT, "NULL argument");
  if (mode < RAP_PLACE_BALANCED || mode > RAP_PLACE_SKEWED) return fail(RAP_ERR_INVALID_ARGUMENT, "bad mode");
  // groups: an output with colocate[j] = i joins i's group (transitively)
  std::vector<int> anchor(n);
  for (int j = 0; j < n; ++j) {
    if (!(cost[j] >= 0)) return fail(RAP_ERR_INVALID_ARGUMENT, "cost must be >= 0");
    const int c = colocate ? colocate[j] : -1;
    if (c >= j || c < -1) return fail(RAP_ERR_INVALID_ARGUMENT, "colocate[j] must be -1 or < j");
    anchor[j] = c < 0 ? j : anchor[c];
  }
  std::vector<int> groups;  // anchors in index order
  std::vector<double> gcost(n, 0.0);
  for (int j = 0; j < n; ++j) {
    if (anchor[j] == j) groups.push_back(j);
    gcost[anchor[j]] += cost[j];
  }
  std::vector<double> load(world, 0.0);
  std::vector<int> gowner(n, 0);
  auto lpt = [&](std::vector<int> gs, int r_lo) {
    std::stable_sort(gs.begin(), gs.end(), [&](int a, int b) { return gcost[a] > gcost[b]; });
    for (int g : gs) {
      int best = r_lo;
      for (int r = r_lo; r < world; ++r)
        if (load[r] < load[best]) best = r;
      gowner[g] = best;
      load[best] += gcost[g];
    }
  };
  if (mode == RAP_PLACE_ROUND_ROBIN) {
    for (size_t i = 0; i < groups.size(); ++i) {
      gowner[groups[i]] = (int)(i % world);
      load[i % world] += gcost[groups[i]];
    }
  } else if (mode == RAP_PLACE_SKEWED && world > 1) {
    double total = 0;
    for (int g : groups) total += gcost[g];
    const double target = 2.0 * total / world;
    std::vector<int> gs = groups, rest;
    std::stable_sort(gs.begin(), gs.end(), [&](int a, int b) { return gcost[a] > gcost[b]; });
    for (int g : gs) {
      if (load[0] + gcost[g] <= target) {
        gowner[g] = 0;
        load[0] += gcost[g];
      } else {
        rest.push_back(g);
      }
    }
    lpt(rest, 1);
  } else {
    lpt(groups, 0);
  }
  for (int j = 0; j < n; ++j) owner_out[j] = gowner[anchor[j]];
  if (residual) {
    residual->output = -1;
    residual->owner = residual->helper = -1;
    residual->pad = 0;
    residual->split_row = n_rows;
    if (world > 1 && n > 0 && n_rows >= 2 * kTileRows) {
      int h = 0, l = 0;
      double total = 0;
      for (int r = 0; r < world; ++r) {
        total += load[r];
        if (load[r] > load[h]) h = r;
        if (load[r] < load[l]) l = r;
      }
      const double mean = total / world;
      if ((comm || load[h] > mean * (1.0 + imbalance_tol)) && h != l) {
        int f = -1;
        for (int j = 0; j < n; ++j)
          if (owner_out[j] == h && (f < 0 || cost[j] > cost[f])) f = j;
        const double per_row = f >= 0 ? cost[f] / (double)n_rows : 0.0;
        if (per_row > 0) {
          double want_rows = 0.5 * (load[h] - load[l]) / per_row;
          double t0 = 0, t1 = 0;  // exchange cost in cost units: t(m) = t0 + m * t1
          if (comm) {
            t0 = comm->link_latency_us / comm->us_per_unit;
            t1 = comm->row_bytes[f] / (1e3 * comm->link_gbs) / comm->us_per_unit;
            want_rows = (load[h] - load[l] - t0) / (2.0 * per_row + t1);
          }
          // split row: a multiple of 128 (whole validity words / tiles on both
          // sides), the owner keeping at least one tile; rounded so that at
          // most want_rows move
          const int64_t want = std::max<int64_t>(0, std::min((int64_t)std::max(0.0, want_rows), n_rows));
          int64_t split = (n_rows - want + kTileRows - 1) / kTileRows * kTileRows;
          split = std::max<int64_t>(split, kTileRows);
          const int64_t moved = n_rows - split;
          bool gain = moved > 0;
          if (comm && gain) {
            const double m = (double)moved;
            const double finish = std::max(load[h] - m * per_row, load[l] + m * per_row + t0 + m * t1);
            gain = finish < load[h];
          }
          if (gain) {
            residual->output = f;
            residual->owner = h;
            residual->helper = l;
            residual->split_row = split;
            load[h] -= per_row * (double)moved;
            load[l] += per_row * (double)moved;
          }
        }
      }
    }
  }
  if (load_out)
    for (int r = 0; r < world; ++r) load_out[r] = load[r];
  return RAP_OK;
}

rap_status rap_plan_create_sharded(const rap_graph* graph, const rap_op_param* params, int32_t n_params, int32_t device,
                                   int32_t sm_budget, const int32_t* sparse_owner, int32_t rank, int32_t world,
                                   rap_plan** out) {
  if (!out) return fail(RAP_ERR_INVALID_ARGUMENT, "out is NULL");
  *out = nullptr;
  if (world < 1 || rank < 0 || rank >= world) return fail(RAP_ERR_INVALID_ARGUMENT, "bad rank/world");
  Validated v;
  rap_status st = validate(graph, params, n_params, &v);
  if (st != RAP_OK) return st;
  std::vector<int32_t> outs;
  int j = 0;
  for (int o = 0; o < graph->n_outputs; ++o) {
    const int node = graph->output_nodes[o];
    if (v.type[node] == VT_IDS) {
      if (!sparse_owner) return fail(RAP_ERR_INVALID_ARGUMENT, "sparse_owner is NULL");
      const int32_t r = sparse_owner[j++];
      if (r < -1 || r >= world) return fail(RAP_ERR_INVALID_ARGUMENT, "sparse_owner out of range");
      if (r == rank) outs.push_back(node);
    } else {
      outs.push_back(node);
    }
  }
  rap_graph g = *graph;
  g.n_outputs = (int32_t)outs.size();
  g.output_nodes = outs.data();
  st = rap_plan_create(&g, params, n_params, device, sm_budget, out);
  if (st != RAP_OK) return st;
  (*out)->rank = rank;
  (*out)->world = world;
  return RAP_OK;
}

rap_status rap_jagged_append(const int32_t* lengths, const int64_t* src_offsets, const int64_t* values, int64_t n,
                             int64_t values_bound, int32_t* dst_lengths, int64_t* dst_offsets, int64_t* dst_values,
                             int64_t dst_capacity, void* stream) {
  if (n < 0 || values_bound < 0 || dst_capacity < 0) return fail(RAP_ERR_INVALID_ARGUMENT, "negative size");
  if (!src_offsets || !dst_offsets) return fail(RAP_ERR_INVALID_ARGUMENT, "offsets NULL");
  if (n > 0 && (!lengths || !dst_lengths)) return fail(RAP_ERR_INVALID_ARGUMENT, "lengths NULL");
  if (values_bound > 0 && (!values || !dst_values)) return fail(RAP_ERR_INVALID_ARGUMENT, "values NULL");
  const int rc = launch_jagged_append(lengths, src_offsets, values, n, values_bound, dst_lengths, dst_offsets,
                                      dst_values, dst_capacity, stream);
  if (rc != 0) return cuda_fail((cudaError_t)rc, "jagged append launch");
  return RAP_OK;
}

// ----------------------------------------------------------------------------
// SM partition (green context, include/rap.h): a stream whose kernels run on
// a dedicated set of SMs (§6.2 L1351-1366 resource-aware sharding,
// enforced by the hardware partition rather than by a CTA-slot cap).  The
// driver entry points are fetched at run time (no libcuda link dependency).
namespace {
struct GreenApi {
  CUresult (*get_dev)(CUdevice*, int) = nullptr;
  CUresult (*get_res)(CUdevice, CUdevResource*, CUdevResourceType) = nullptr;
  CUresult (*split)(CUdevResource*, unsigned int*, const CUdevResource*, CUdevResource*, unsigned int,
                    unsigned int) = nullptr;
  CUresult (*gen_desc)(CUdevResourceDesc*, CUdevResource*, unsigned int) = nullptr;
  CUresult (*create)(CUgreenCtx*, CUdevResourceDesc, CUdevice, unsigned int) = nullptr;
  CUresult (*destroy)(CUgreenCtx) = nullptr;
  CUresult (*stream_create)(CUstream*, CUgreenCtx, unsigned int, int) = nullptr;
  CUresult (*stream_destroy)(CUstream) = nullptr;
  bool ok = false;
};
const GreenApi& green_api() {
  static GreenApi g;
  static std::once_flag once;
  std::call_once(once, [] {
    auto get = [](const char* name, void** fn) {
      cudaDriverEntryPointQueryResult q;
      return cudaGetDriverEntryPoint(name, fn, cudaEnableDefault, &q) == cudaSuccess &&
             q == cudaDriverEntryPointSuccess && *fn != nullptr;
    };
    g.ok = get("cuDeviceGet", reinterpret_cast<void**>(&g.get_dev)) &&
           get("cuDeviceGetDevResource", reinterpret_cast<void**>(&g.get_res)) &&
           get("cuDevSmResourceSplitByCount", reinterpret_cast<void**>(&g.split)) &&
           get("cuDevResourceGenerateDesc", reinterpret_cast<void**>(&g.gen_desc)) &&
           get("cuGreenCtxCreate", reinterpret_cast<void**>(&g.create)) &&
           get("cuGreenCtxDestroy", reinterpret_cast<void**>(&g.destroy)) &&
           get("cuGreenCtxStreamCreate", reinterpret_cast<void**>(&g.stream_create)) &&
           get("cuStreamDestroy", reinterpret_cast<void**>(&g.stream_destroy));
  });
  return g;
}
std::mutex g_green_mu;
std::map<void*, CUgreenCtx>* g_green = nullptr;  // stream -> its green context
}  // namespace

extern "C" {

rap_status rap_sm_partition_stream(int32_t device, int32_t n_sms, int32_t priority, void** stream_out,
                                   int32_t* sms_out) {
  if (!stream_out || n_sms < 1) return fail(RAP_ERR_INVALID_ARGUMENT, "stream_out NULL or n_sms < 1");
  *stream_out = nullptr;
  const GreenApi& g = green_api();
  if (!g.ok) return fail(RAP_ERR_UNSUPPORTED, "green-context driver entry points unavailable");
  DeviceGuard dg(device);
  cudaFree(nullptr);  // the runtime's primary context exists (driver initialised)
  CUdevice dev;
  if (g.get_dev(&dev, device) != CUDA_SUCCESS) return fail(RAP_ERR_CUDA, "cuDeviceGet");
  CUdevResource all, part, rest;
  if (g.get_res(dev, &all, CU_DEV_RESOURCE_TYPE_SM) != CUDA_SUCCESS) return fail(RAP_ERR_CUDA, "cuDeviceGetDevResource");
  if ((unsigned)n_sms >= all.sm.smCount) return fail(RAP_ERR_INVALID_ARGUMENT, "n_sms >= the device's SMs");
  unsigned int groups = 1;
  // one group of at least n_sms SMs (sm_100: multiples of 8, at least 8)
  if (g.split(&part, &groups, &all, &rest, 0, (unsigned)n_sms) != CUDA_SUCCESS || groups < 1)
    return fail(RAP_ERR_CUDA, "cuDevSmResourceSplitByCount");
  CUdevResourceDesc desc;
  if (g.gen_desc(&desc, &part, 1) != CUDA_SUCCESS) return fail(RAP_ERR_CUDA, "cuDevResourceGenerateDesc");
  CUgreenCtx gctx;
  if (g.create(&gctx, desc, dev, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS) return fail(RAP_ERR_CUDA, "cuGreenCtxCreate");
  CUstream st;
  if (g.stream_create(&st, gctx, CU_STREAM_NON_BLOCKING, priority) != CUDA_SUCCESS) {
    g.destroy(gctx);
    return fail(RAP_ERR_CUDA, "cuGreenCtxStreamCreate");
  }
  {
    std::lock_guard<std::mutex> lk(g_green_mu);
    if (!g_green) g_green = new std::map<void*, CUgreenCtx>();
    (*g_green)[reinterpret_cast<void*>(st)] = gctx;
  }
  *stream_out = reinterpret_cast<void*>(st);
  if (sms_out) *sms_out = (int32_t)part.sm.smCount;
  return RAP_OK;
}

rap_status rap_sm_partition_stream_destroy(void* stream) {
  const GreenApi& g = green_api();
  CUgreenCtx gctx = nullptr;
  {
    std::lock_guard<std::mutex> lk(g_green_mu);
    if (!g_green || !g_green->count(stream)) return fail(RAP_ERR_INVALID_ARGUMENT, "not a partition stream");
    gctx = (*g_green)[stream];
    g_green->erase(stream);
  }
  g.stream_destroy(reinterpret_cast<CUstream>(stream));
  g.destroy(gctx);
  return RAP_OK;
}

}  // extern "C"
