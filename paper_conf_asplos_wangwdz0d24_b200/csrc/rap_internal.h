// rap_internal.h — device program format shared by the host planner
// (rap_plan.cpp) and the fused kernel (rap_kernel.cu).  Product code only;
// nothing here is shared with oracle/.
//
// A plan lowers every output of the preprocessing DAG to
// a flattened, position-independent program that a CTA copies into shared
// memory in one coalesced burst before it processes a descriptor:
//  - SProg, one per sparse output: an id-list chain (source = raw sparse
//    column, dense expression + Bucketize, or NGram over up to 8 source
//    chains), elementwise id ops, FirstX folded into a length cap and FillNull
//    into a null-row rule, plus an optional staged Bucketize border table;
//  - DProg, one per dense column group: the dense expressions and OneHot
//    units that produce up to kGroupCols adjacent output columns.
// DESIGN.md §7 describes the layout.
#pragma once
#ifdef __CUDACC_RTC__
// NVRTC (the plan-specialised kernel, rap_jit.cpp): no system headers
typedef signed char int8_t;
typedef short int16_t;
typedef int int32_t;
typedef long long int64_t;
typedef unsigned char uint8_t;
typedef unsigned short uint16_t;
typedef unsigned int uint32_t;
typedef unsigned long long uint64_t;
typedef unsigned long long uintptr_t;
#define INT32_MAX 2147483647
#define INT64_MAX 9223372036854775807LL
#define INT64_MIN (-INT64_MAX - 1LL)
#else
#include <stdint.h>
#include <stdlib.h>
#endif

#ifdef __CUDACC__
#define RAP_HD __host__ __device__ __forceinline__
#else
#define RAP_HD inline
#endif

namespace rapk {

constexpr int kThreads = 256;          // threads per CTA
constexpr int kMaxNgramK = 8;          // NGram sources (R7: 1 <= k <= 8)
constexpr int64_t kNoCap = INT64_MAX;
constexpr int kVBuf = 2048;            // output ids a sparse descriptor stages in smem
constexpr int kRowsSparseMax = 1024;   // rows per sparse descriptor (upper bound)
constexpr int kNgSlots = 1024;         // NGram (source, row) slots per descriptor: k * rows <= kNgSlots
constexpr int kMaxStagedOps = 32;      // ops carried inside an SProg
constexpr int kStageTab = 1024;        // int64 Bucketize borders staged with an SProg
constexpr int kGroupCols = 64;         // dense output columns per column group
constexpr int kMaxDenseOps = 96;       // ops carried inside a DProg
constexpr int kDenseTabF = 256;        // f32 borders carried inside a DProg
constexpr int kDenseTileBytes = 28672; // dense row-major tile budget (smem)
constexpr int kDenseInBytes = 12288;   // dense input columns staged per descriptor (smem)
constexpr int kInVals = 2048;          // child ids of a sparse descriptor staged in smem
constexpr int kInOff = 1088;           // staged offsets (all sources of a descriptor)
constexpr int kInBm = 128;             // staged validity words (all sources)

// Elementwise op kinds.  Dense ops act on an f32 scalar, id ops on int64.
enum OpKind : int32_t {
  OK_FILL_F = 0,    // dense FillNull: NaN -> f0                                  (R10)
  OK_LOGIT = 1,     // f0 = lo = eps, f1 = hi = 1 - eps (f32)                     (R11)
  OK_BOXCOX = 2,    // f0 = lambda                                                (R12)
  OK_CLAMP = 3,     // a = lo, b = hi                                             (R6)
  OK_SIGRID = 4,    // hsalt = H(salt), M                                         (R3)
  OK_BUCKET_I = 5,  // global itab[a .. a+m) sorted int64 borders                 (R4)
  OK_MAPID = 6,     // open-addressing table of 2^m (key, val) slots at itab[a ..),
                    // b = default, M = 1 if INT64_MIN is a key (its value in hsalt) (R8)
  OK_BUCKET_S = 7   // borders staged with the program: table[a .. a+m)          (R4)
};

struct DevOp {
  int32_t kind, m;
  int64_t a, b;
  uint64_t hsalt;
  int64_t M;
  float f0, f1;
};

enum SrcKind : int32_t { SRC_SPARSE = 0, SRC_DENSE_BUCKET = 1, SRC_NGRAM = 2 };

// Id-list chain (op indices are local to the program that holds it).
// Valid rows: out = ops[op_begin,op_end)(src[j]) for j < min(L, xcap).
// Null rows of a SRC_SPARSE source: with has_fill the list is [fill] passed
// through ops[null_op_begin, op_end) and capped at null_xcap, otherwise empty
// (R14).  SRC_DENSE_BUCKET: src = raw dense column, dense ops
// [dop_begin, dop_end), f32 borders ftab[btab .. btab+bm) (global).
struct Chain {
  int32_t src_kind, src;
  int32_t op_begin, op_end;
  int32_t null_op_begin, has_fill;
  int64_t xcap, null_xcap;
  int64_t fill;
  int32_t btab, bm;
  int32_t dop_begin, dop_end;
};

struct NGramDesc {
  int32_t n, k;
  uint64_t hsalt;  // H(salt)
  int64_t M;
  int32_t chain[kMaxNgramK];  // host-side chain indices (unused on the device)
};

// Canonical pipeline: a SRC_SPARSE chain whose id ops are an
// ordered subset of Clamp -> MapId -> SigridHash -> Bucketize (each at most
// once, MapId without an INT64_MIN key) runs through a specialised,
// register-resident code path instead of the op interpreter.  mask bits:
// 1 Clamp, 2 MapId, 4 SigridHash, 8 Bucketize; null_mask = the stages a
// filled null row goes through.  For an NGram output the same form describes
// the post-hash ops.
enum CanonBit : int32_t { CB_CLAMP = 1, CB_MAPID = 2, CB_SIGRID = 4, CB_BUCKET = 8 };
struct Canon {
  int32_t ok, mask, null_mask, map_m;
  int32_t bk_m, pad;
  int64_t lo, hi;          // Clamp
  int64_t map_a, map_def;  // MapId: itab offset of the table, default
  uint64_t hs;             // SigridHash: H(salt)
  int64_t M;
  int64_t bk_a;            // Bucketize: absolute itab offset of the borders
};

struct SProg {
  Chain ch;
  Chain src[kMaxNgramK];
  NGramDesc ng;
  Canon cn;                  // the output chain (post-hash ops for an NGram)
  Canon src_cn[kMaxNgramK];  // NGram sources
  int32_t n_ops;       // ops used
  int32_t tab_len;     // staged int64 table entries (OK_BUCKET_S)
  int32_t global_ops;  // 1: op indices refer to Common::ops (program too large to stage)
  int32_t pad;
  int64_t tab_off;     // itab offset of the staged table
  DevOp ops[kMaxStagedOps];
};

enum UnitKind : int32_t { U_DENSE = 0, U_ONEHOT_DB = 1, U_ONEHOT_G = 2 };

// A dense output unit of a column group: one Dense column (U_DENSE), or the
// columns [col, col+width) of a OneHot holding ids [k0, k0+width) —
// U_ONEHOT_DB when its list is a dense Bucketize (id ops [iop_begin, iop_end),
// cap xcap), U_ONEHOT_G (any other list) through the SProg oprogs[prog].
// gops = 1: op indices / borders refer to Common::ops / Common::ftab.
// slot: index of src_col in DProg::cols (the staged input columns).
struct DUnit {
  int32_t kind, col, width, src_col;
  int32_t op_begin, op_end;
  int32_t btab, bm;
  int32_t iop_begin, iop_end;
  int32_t prog, gops;
  int32_t slot, pad;
  int64_t k0, xcap;
};

struct DProg {
  int32_t n_units, width, col0, any_onehot;
  int32_t n_ops, n_ftab, n_cols, pad1;
  int32_t cols[kGroupCols];  // distinct raw dense columns read by the group
  DUnit units[kGroupCols];
  DevOp ops[kMaxDenseOps];
  float ftab[kDenseTabF];
};

// Work decomposition of one launch.  Units are the sparse
// tiles (output f, 128-row range rt), numbered feature-major t = f * T + rt
// (the order of the jagged scan, R17), followed by the dense blocks (128 rows
// x one column group).  The host splits the unit sequence into one
// contiguous, cost-balanced range per CTA (Common::part); a CTA sums its
// sparse tiles' output lengths, publishes that aggregate, runs its dense
// blocks, adds its predecessors' aggregates and then writes its tiles.  No
// grid barrier, no per-tile look-back.
constexpr int kMaxCtas = 2048;        // grid cap
constexpr int kWarpsPerCta = kThreads / 32;
constexpr int kPartLen = kMaxCtas * kWarpsPerCta + 1;  // per-warp partition boundaries
constexpr int kPartSlots = 8;         // cached partitions per plan
constexpr int kTileRows = 128;        // rows of a sparse tile (4 groups of 32)
constexpr int kDenseBlockRows = 128;  // rows of a dense block (CTA unit)

// Non-array kernel parameters.
struct Common {
  const SProg* sprogs;        // [n_sparse_out]
  const SProg* oprogs;        // OneHot generic programs
  const DProg* dprogs;        // [n_groups]
  const DevOp* ops;           // global op array (programs too large to stage)
  const float* ftab;
  const int64_t* itab;
  int32_t n_sparse_out, n_groups;
  int64_t n_rows;
  int64_t tiles_per_feature;  // T = ceil(n_rows / kTileRows)
  int64_t n_sparse_tiles;     // S = n_sparse_out * T
  int64_t n_dense_tiles;      // n_groups * ceil(n_dense_rows / kDenseBlockRows)
  int64_t dense_row0;         // dense outputs cover raw rows [dense_row0, dense_row0 + n_dense_rows)
  int64_t n_dense_rows;       // (a sharded plan's batch shard; else 0 and n_rows)
  int32_t chain;              // 1: offsets/value positions start at offsets[0] (rap_output RAP_OUT_CHAIN)
  int32_t vi32;               // 1: values are int32 (rap_output RAP_OUT_VALUES_I32, Cast)
  // sched[0] = CTAs done, sched[1] = launch epoch; the last CTA resets the
  // counter and advances the epoch, so launch parameters are identical from
  // call to call (CUDA-graph replayable).
  unsigned long long* sched;
  const int64_t* part;         // [grid * 8 + 1] unit range of each warp (CTA rank r: slots 8r .. 8r+8)
  unsigned long long* agg;     // [kMaxCtas] per-rank aggregate words (epoch-tagged)
  float* dense_out;
  int64_t ld;
  int32_t* lengths;
  int64_t* offsets;
  int64_t* values;
  int64_t values_cap;
  int32_t* err;
  // profiling aid (rap_debug_trace): kTracePts globaltimer stamps per CTA
  unsigned long long* trace;
  int64_t trace_cap;
};

constexpr int kTracePts = 24;

struct LaunchRaw {
  int32_t n_dense, n_sparse;
  const float* const* dense;
  const uint32_t* const* dvalid;
  const int32_t* const* off;
  const int64_t* const* val;
  const uint32_t* const* svalid;
};

// ---- hash (reading R1/R2), product-side implementation ----
RAP_HD uint64_t splitmix_H(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// ---- Row-block kernel (rap_rows.cu) ----
// The batch's rows are split into n_rb contiguous row blocks and the sparse
// outputs into n_fg feature groups; CTA (g, r) evaluates group g over block
// r, one row per thread, in 256-row chunks: (1) output lengths from the Arrow
// offsets staged in shared memory, summed per output into agg[f * n_rb + r]
// and announced on a release counter; (2) dense blocks; (3) the base of every
// output of the group = the feature-major exclusive prefix of those totals
// (warp-parallel reductions); (4) lengths, offsets and ids.
constexpr int kRbChunk = 256;   // rows per chunk (one per thread)
constexpr int kRbMaxFg = 64;    // feature groups
constexpr int kRbMaxFL = 64;    // sparse outputs per feature group (interpreted form)
constexpr int kJitMaxF = 192;   // sparse outputs of the generated kernel's one group (<= its 224 sparse threads)
constexpr int kRbMaxF = 1024;   // sparse outputs of a plan the row-block kernel takes
constexpr int kRbMaxCols = 64;  // raw sparse columns the row-block kernel addresses
constexpr int kRbMaxDense = 32; // raw dense columns
constexpr int kRbPitchPairs = 132;  // staged offsets per column in warp-pair mode (128-row chunks)
constexpr int kRbIdCap = 232;   // staged ids per column and chunk (224 rows of single ids + 16-byte head/tail)

// Per sparse output (indexed by output f): its closed-form length program
// (R5, R7, R10, R14 from the Arrow offsets and validity bits of up to
// kMaxNgramK raw columns) and how its ids are emitted.
//   kind 0: one list source; 1: constant (a dense Bucketize, R4); 2: NGram.
//   emit 0: canonical list (Canon stages), 1: generic list, 2: dense bucket,
//        3: NGram.
// Memo: a canonical list output saves element 0 of each row after the stages
// in memo_mask into shared slot memo_slot, and an NGram source k whose chain
// is that prefix reads it (prov[k] = the provider's processing index, so
// the kernel uses it only if the provider ran earlier in the same CTA).
struct RbFeat {
  int32_t kind, n, k, out_cap;  // out_cap: NGram FirstX cap, or kind 1's constant
  int32_t src[kMaxNgramK];      // raw sparse column, -1 = dense-bucket source (length cap[i])
  int32_t cap[kMaxNgramK];      // FirstX cap of a valid row
  int32_t ncap[kMaxNgramK];     // length of a null row (filled: min(1, cap), else 0)
  int32_t emit, memo_slot, memo_mask, pad;
  int32_t prov[kMaxNgramK];
  int32_t pslot[kMaxNgramK];
};

constexpr int kRbSup = 32;                  // row blocks per super block (two-level lower-block sums)
constexpr int kRbSupMax = kMaxCtas / kRbSup;  // super blocks per output
struct RbGeom {
  int32_t n_rb, n_fg, rows_rb, max_fl;  // row blocks, feature groups, rows per block (x32), max outputs per group
  int32_t max_cols, dense_bytes;        // max raw sparse columns one group stages; dense-phase smem bytes
  int32_t n_memo, small;                // memo slots; small = 1: every base fits 31 bits (32-bit scans)
  int32_t len_cache;                    // 1: the kernel keeps a uint16 length cache per (output, row) in smem
  int32_t n_dcta;                       // dedicated dense CTAs after the n_rb x n_fg sparse ones (0: dense
                                        // blocks round robin over every CTA)
  int32_t id_slots;                     // staged columns (slots < id_slots) whose chunk ids are bulk-copied
                                        // into shared memory (generated kernel; 0: ids read from global)
  int32_t pitch;                        // staged offsets per column (0: kRbPitch, 256-row chunks)
  int32_t feat_recs;                    // 1: the CTA keeps RbF records in shared memory (interpreter)
  unsigned long long all_cols;          // raw sparse columns the outputs read (bit c: column c < 64)
  const RbFeat* feat;                   // [n_sparse_out], by output index
  const int32_t* perm;                  // [n_sparse_out] processing order (groups are ranges of it)
  unsigned long long* agg;              // [n_sparse_out][n_rb] per-(output, row block) totals
  unsigned long long* sched;            // [0] CTAs done, [2] CTAs whose totals are stored (reset by the last CTA)
  unsigned long long* tot;              // [n_sparse_out] per-output totals (red.add; zeroed by the last CTA)
  unsigned long long* sup;              // [n_sparse_out][kRbSupMax] totals of 32-row-block super blocks (red.add)
  int32_t fg_off[kRbMaxFg + 1];         // group g = perm[fg_off[g] .. fg_off[g + 1])
};

// Launch entry implemented in rap_kernel.cu (cooperative launch: every CTA
// is resident, so a CTA may wait on its predecessors' aggregates).
// Returns a cudaError_t value.
int launch_fused(const Common& c, const LaunchRaw& raw, int grid, int smem_bytes, void* stream);
// Dynamic shared memory per CTA for dense groups up to max_width columns.
int fused_smem_bytes(int max_width);
// rap_jagged_append's kernel (rap_kernel.cu).
int launch_jagged_append(const int32_t* len, const int64_t* so, const int64_t* val, int64_t n, int64_t vb, int32_t* dl,
                         int64_t* dof, int64_t* dv, int64_t cap, void* stream);
// One launch copying n device-mapped pinned host ranges into device buffers (rap_kernel.cu).
int launch_gather_h2d(const void* const* src, void* const* dst, const int64_t* bytes, int n, void* stream);
// Exact-size copy of values[0, *total) into device-mapped pinned host memory (rap_kernel.cu).
int launch_values_to_host(const int64_t* src, const int64_t* total, int64_t cap, int64_t* dst, void* stream);
// Raise a kernel's MaxDynamicSharedMemorySize on the current device to at
// least smem (never lowers it: plans of different geometries share the kernel,
// so an attribute set for one plan must stay valid for every other).  One
// process-wide record per (kernel, device), mutex-guarded.  rap_kernel.cu.
int ensure_dyn_smem(const void* kernel, int smem);
// Occupancy query: CTAs per SM for the given dynamic smem.
int fused_occupancy(int smem_bytes, int n_dense, int n_sparse, int* ctas_per_sm);
// Row-block kernel (rap_rows.cu): dynamic smem for a geometry, occupancy, launch.
int rows_smem_bytes(int dense_bytes, int max_fl, int max_cols, int n_memo, int n_sparse_out, int len_cache,
                    int id_slots = 0, int pitch = 0, int feat_recs = 1, int tab_bytes = 0);
// Dense-phase shared memory of the row-block kernel for dense groups up to max_width columns.
int rows_dense_bytes(int max_width);
int rows_occupancy(int smem_bytes, int* ctas_per_sm);
int launch_rows(const Common& c, const RbGeom& g, const LaunchRaw& raw, int smem_bytes, void* stream);

#ifndef __CUDACC_RTC__
// ---- Plan-specialised row-block kernel (rap_jit.cpp) ----
// The planner's view of a plan that the code generator reads.
struct JitPlanView {
  int n_sparse_out, n_sparse_in;
  const RbFeat* feat;    // [n_sparse_out]
  const SProg* sprogs;   // [n_sparse_out]
  const int32_t* perm;   // [n_sparse_out] processing order
  const int* used_sparse;
  int n_used_sparse;
  // dense outputs (DProg column groups, rap_internal.h)
  const DProg* dprogs;
  int n_dprogs, d_out, dense_bytes;  // dense_bytes: the kernel's dense-phase shared memory
  const int64_t* itab;               // the plan's int64 table pool (Bucketize borders, MapId tables)
  const DevOp* ops;                  // global op pool (DUnit::gops = 1: units too large to stage)
  const float* ftab;                 // global f32 border pool (DUnit::gops = 1)
  int id_slots;                      // staged slots whose ids the kernel stages in shared memory (RbGeom)
  int pairs;                         // warp-pair mode (rap_rows_skel.cuh kPairs)
};
struct JitModule;  // compiled kernels (opaque)
// How the generated kernel evaluates the dense outputs (rap_jit.cpp):
//   2: every warp evaluates 32-row tiles of its block's dense rows (one
//      row-major tile per warp in shared memory) after the block's totals
//      are published, so the work fills the wait for the other CTAs;
//   1: one dense warp (warp 7) beside the sparse phases (tiles too wide for
//      eight per CTA);
//   0: no generated dense code (the interpreted dense blocks).
// *region0 = the shared-memory bytes of region 0 the mode needs.
//   3: three dense warps (warps 7-9 of a 320-thread CTA) beside the sparse
//      phases, each with its own tile: the dense work overlaps the emit
//      phase, whose warps leave most issue slots idle (the default).
inline int jit_dense_tiles(int) { return 8; }  // mode 2: warps with a tile
#ifndef __CUDACC_RTC__
inline int jit_dense_warps3() {  // mode 3's dense warps (RAP_JIT_DENSE_WARPS: experiment knob, read once)
  static const int n = [] {
    const char* e = getenv("RAP_JIT_DENSE_WARPS");
    const int v = e ? atoi(e) : 3;
    return v < 1 ? 1 : (v > 8 ? 8 : v);
  }();
  return n;
}
#else
inline int jit_dense_warps3() { return 3; }
#endif
inline int jit_dense_warps(int mode) { return mode == 3 ? jit_dense_warps3() : mode == 1 ? 1 : 0; }
inline int jit_dense_mode(int n_sparse_out, int d_out, int n_dprogs, int rb_dense_bytes, int pairs, int* region0) {
  const int off = ((2 * (n_sparse_out + 1) * 8) + 15) & ~15;  // after the base phase's T[f], L[f]
  const int one = 32 * (d_out | 1) * 4;
  const int nt = jit_dense_tiles(pairs);
  if (n_dprogs == 0 || d_out <= 0) {
    *region0 = rb_dense_bytes;
    return 0;
  }
#ifndef __CUDACC_RTC__
  static const int wm = [] {  // "1" / "2": force that mode (experiment knob; read once per process)
    const char* want = getenv("RAP_JIT_DENSE");
    return want ? atoi(want) : 3;
  }();
#else
  const int wm = 3;
#endif
  if (wm == 3 && !pairs && off + jit_dense_warps3() * one <= 48 * 1024) {
    *region0 = off + jit_dense_warps3() * one;
    return 3;
  }
  if (wm != 1 && off + nt * one <= 48 * 1024) {
    *region0 = off + nt * one;
    return 2;
  }
  if (pairs) {  // the warp-pair form has no dense warp: interpreted dense blocks
    *region0 = rb_dense_bytes;
    return 0;
  }
  (void)wm;
  if (off + one <= rb_dense_bytes) {
    *region0 = off + one;
    return 1;
  }
  *region0 = rb_dense_bytes;
  return 0;
}
// Generate the CUDA source of the plan's policy (small: 32-bit scans, every
// offset < 2^31; else 64-bit) and compile it with NVRTC for sm_100a (cached
// per source text in the process).  Returns nullptr and fills *log on failure.
JitModule* jit_build(const JitPlanView& v, int variant, char* log, int log_cap);  // bit 0 small, bit 1 int32 values
int jit_occupancy(JitModule* m, int smem_bytes, int threads, int* ctas_per_sm);
// Region-0 shared-memory bytes the generated kernel needs beyond the dense
// tile (the column emitter's memo rows; 0 if none).
int jit_dense_need(const JitPlanView& v);
// Shared-memory bytes of the tables the generated kernel stages at launch
// (Bucketize borders and sub-block maxima; 0: none).
int jit_table_bytes(const JitPlanView& v);
int launch_jit(JitModule* m, const Common& c, const RbGeom& g, const LaunchRaw& raw, int smem_bytes, int threads,
               void* stream);
double jit_compile_seconds(const JitModule* m);
#endif
}  // namespace rapk
#if !defined(__CUDACC_RTC__) && defined(__cplusplus)
#include <string>
namespace rapk {
std::string jit_generate(const JitPlanView& v);
bool jit_compile_only(const std::string& src, std::string* log);
}  // namespace rapk
#endif
namespace rapk {

}  // namespace rapk
