// rap_internal.h — device program format shared by the host planner
// (rap_plan.cpp) and the fused kernel (rap_kernel.cu).  Product code only;
// nothing here is shared with oracle/.
//
// A plan lowers every output of the preprocessing DAG to
// a small "op program": a source (raw sparse column, dense expression then
// Bucketize, or NGram) followed by elementwise id ops, with FirstX folded into
// a length cap and FillNull into a null-row rule.
#pragma once
#include <stdint.h>

#ifdef __CUDACC__
#define RAP_HD __host__ __device__ __forceinline__
#else
#define RAP_HD inline
#endif

namespace rapk {

constexpr int kThreads = 256;        // threads per CTA
constexpr int kMaxNgramK = 8;        // NGram sources (R7: 1 <= k <= 8)
constexpr int64_t kNoCap = INT64_MAX;

// Elementwise op kinds.  Dense ops act on an f32 scalar, id ops on int64.
enum OpKind : int32_t {
  OK_FILL_F = 0,   // dense FillNull: NaN -> f0                          (R10)
  OK_LOGIT = 1,    // f0 = lo = eps, f1 = hi = 1 - eps (f32)            (R11)
  OK_BOXCOX = 2,   // f0 = lambda                                        (R12)
  OK_CLAMP = 3,    // a = lo, b = hi                                     (R6)
  OK_SIGRID = 4,   // hsalt = H(salt), M                                 (R3)
  OK_BUCKET_I = 5, // itab[a .. a+m) sorted int64 borders                (R4)
  OK_MAPID = 6     // itab[a .. a+m) sorted keys, itab[a+m ..) vals, b = default (R8)
};

struct DevOp {
  int32_t kind, m;
  int64_t a, b;
  uint64_t hsalt;
  int64_t M;
  float f0, f1;
};

enum SrcKind : int32_t { SRC_SPARSE = 0, SRC_DENSE_BUCKET = 1, SRC_NGRAM = 2 };

// Dense expression: raw dense column -> ops[op_begin, op_end) (all dense ops).
struct DenseExpr {
  int32_t col, op_begin, op_end, pad;
};

// Id-list chain.  Valid rows: out = ops[op_begin,op_end)(src[j]) for
// j < min(L, xcap).  Null rows of a SRC_SPARSE source: if has_fill the list
// is [fill] passed through ops[null_op_begin, op_end) and capped at
// null_xcap, otherwise empty (R14).
struct Chain {
  int32_t src_kind, src;        // sparse column | dense expr | ngram index
  int32_t op_begin, op_end;
  int32_t null_op_begin, has_fill;
  int64_t xcap, null_xcap;
  int64_t fill;
  int32_t btab, bm;             // SRC_DENSE_BUCKET: f32 borders ftab[btab .. btab+bm)
};

struct NGramDesc {
  int32_t n, k;
  uint64_t hsalt;               // H(salt)
  int64_t M;
  int32_t chain[kMaxNgramK];
};

enum UnitKind : int32_t { U_DENSE = 0, U_ONEHOT = 1 };

// A dense output unit inside a column group: one Dense column, or the
// columns [col, col+width) of a OneHot, holding ids [k0, k0+width).
struct Unit {
  int32_t kind, idx, col, width;
  int64_t k0;
};

// Column group: the dense output columns [col0, col0+width) one dense
// descriptor writes for its row block.
struct Group {
  int32_t unit_begin, unit_end, col0, width;
};

struct SparseOut {
  int32_t chain, rows_per_desc;
};

// Non-array kernel parameters.
struct Common {
  const DevOp* ops;
  const DenseExpr* dexprs;
  const Chain* chains;
  const NGramDesc* ngrams;
  const Unit* units;
  const Group* groups;
  const SparseOut* souts;
  const float* ftab;
  const int64_t* itab;
  const int32_t* desc_start;    // [n_sparse_out + 1] for this n_rows
  int32_t n_sparse_out, n_groups, rows_dense, tile_ld;
  int64_t n_rows, n_sparse_desc, n_total_desc;
  // sched[0] = ticket counter, sched[1] = CTAs done, sched[2] = epoch.  The
  // last CTA to finish resets the counters and advances the epoch, so the
  // launch parameters are identical from call to call (CUDA-graph replayable).
  unsigned long long* sched;
  unsigned long long* status;   // decoupled look-back words, one per sparse descriptor
  int64_t status_cap;
  float* dense_out;
  int64_t ld;
  int32_t* lengths;
  int64_t* offsets;
  int64_t* values;
  int64_t values_cap;
  int32_t* err;
};

struct LaunchRaw {
  int32_t n_dense, n_sparse;
  const float* const* dense;
  const uint32_t* const* dvalid;
  const int32_t* const* off;
  const int64_t* const* val;
  const uint32_t* const* svalid;
};

// Status word of the look-back: [63:44] epoch, [43:42] flag, [41:0] value.
constexpr int kEpochShift = 44;
constexpr int kFlagShift = 42;
constexpr unsigned long long kValueMask = (1ull << 42) - 1;
constexpr unsigned long long kFlagAgg = 1, kFlagPrefix = 2;
constexpr unsigned long long kEpochMax = (1ull << 20) - 1;

// ---- hash (reading R1/R2), product-side implementation ----
RAP_HD uint64_t splitmix_H(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Launch entry implemented in rap_kernel.cu.  Returns a cudaError_t value.
int launch_fused(const Common& c, const LaunchRaw& raw, int grid, int smem_bytes, void* stream);
// Occupancy query: CTAs per SM for the given dynamic smem.
int fused_occupancy(int smem_bytes, int n_dense, int n_sparse, int* ctas_per_sm);

}  // namespace rapk
