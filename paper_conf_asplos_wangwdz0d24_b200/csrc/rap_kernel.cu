// rap_kernel.cu — the fused, persistent sm_100a preprocessing kernel.
//
// One launch processes a whole raw batch (§6.1:
// horizontal fusion of the per-feature kernels; here every op of every
// feature runs in one persistent kernel, so the chains are fused vertically
// as well and no intermediate touches HBM).  The jagged offsets are a global
// exclusive scan over (feature, row) in feature-major order (R17), done in a
// single pass with a decoupled look-back:
//   (1) warps take 128-row sparse tiles from a global queue in scan order;
//       a tile computes its output lengths (closed form from the Arrow
//       offsets and validity words), publishes their sum, computes its ids
//       (base-independent), resolves its base from its predecessors' words,
//       then stores lengths, offsets and ids;
//   (2) CTAs take dense column-group blocks from a second queue (inputs
//       staged by cp.async.bulk onto an mbarrier, evaluated (row, unit)-
//       parallel into a row-major smem tile, float4 stores).
// No grid barrier and no cross-CTA wait other than the look-back; queue
// order = scan order, so a tile only ever waits on tiles already taken.  The
// grid is capped by the SM budget (§6.2).
//
// Operator semantics: DESIGN.md §3 readings R1-R20 (Table 1).
// Nothing here is tensor-core work: the path is integer ALU + a few SFU
// transcendentals, bound by HBM bandwidth and issue.
#include <cuda_runtime.h>
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#include <string.h>

#include "rap_internal.h"

namespace rapk {

template <int MD, int MS>
struct KParams {
  Common c;
  const float* dense[MD];
  const uint32_t* dvalid[MD];
  const int32_t* off[MS];
  const int64_t* val[MS];
  const uint32_t* svalid[MS];
};

constexpr int kWarps = kThreads / 32;
constexpr int kGroups = kTileRows / 32;  // row groups of a sparse tile (one row per lane each)
constexpr int kNgScratch = kWarps * 4 * kMaxNgramK * 32 * 4;  // NGram warp scratch (smem, sparse phase)
// Look-back word: [63:44] epoch, [43:42] flag, [41:0] value.
constexpr int kEpochShift = 44;
constexpr int kFlagShift = 42;
constexpr unsigned long long kValueMask = (1ull << 42) - 1;
constexpr unsigned long long kFlagAgg = 1, kFlagPrefix = 2;
constexpr unsigned long long kEpochMax = (1ull << 20) - 1;

__host__ __device__ constexpr int align_up(int x, int a) { return (x + a - 1) / a * a; }

// ----------------------------------------------------------------------------
// Scalar helpers.

__device__ __forceinline__ uint64_t reduce_M(uint64_t h, int64_t M) {  // R2
  return __umul64hi(h, (uint64_t)M);
}

__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

// Profiling aid: per-CTA phase stamps (%globaltimer), thread 0 only, enabled
// when the plan allocated a trace buffer (rap_debug_trace).
__device__ __forceinline__ void trace_stamp(const Common& c, int k) {
  if (c.trace != nullptr && threadIdx.x == 0 && (int64_t)blockIdx.x < c.trace_cap) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    c.trace[(int64_t)blockIdx.x * kTracePts + k] = v;
  }
}

// ---- mbarrier + bulk async copies (TMA engine, non-tensor form) ----
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "RAP_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra RAP_WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}

// bytes: multiple of 16; dst, src: 16-byte aligned.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_relaxed(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ long long warp_sum64(long long v) {
#pragma unroll
  for (int d = 16; d >= 1; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
  return v;
}

// Upper bound = #{i : b[i] <= x} for sorted borders (R4; NaN -> 0).
template <class T>
__device__ __forceinline__ int64_t upper_bound(const T* b, int m, T x) {
  int lo = 0, n = m;
  while (n > 0) {
    const int half = n >> 1;
    if (__ldg(b + lo + half) <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}

__device__ __forceinline__ int64_t upper_bound_s(const float* b, int m, float x) {  // shared-memory borders
  int lo = 0, n = m;
  while (n > 0) {
    const int half = n >> 1;
    if (b[lo + half] <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}

// MapId (R8) through an open-addressing table built by the planner:
// 2^m slots of (key, value), empty key = INT64_MIN, Fibonacci hashing,
// linear probing.  A real INT64_MIN key is carried in the op (M = 1, hsalt).
__device__ __forceinline__ int64_t map_lookup(const int64_t* itab, int64_t a, int m, int64_t dflt, int has_min,
                                              int64_t min_val, int64_t x) {
  if (x == INT64_MIN) return has_min ? min_val : dflt;
  const longlong2* t = reinterpret_cast<const longlong2*>(itab + a);
  const uint32_t mask = (1u << m) - 1u;
  uint32_t i = (uint32_t)(((uint64_t)x * 0x9E3779B97F4A7C15ull) >> (64 - m));
  while (true) {
    const longlong2 kv = __ldg(t + i);
    if (kv.x == x) return kv.y;
    if (kv.x == INT64_MIN) return dflt;
    i = (i + 1) & mask;
  }
}

// One id op; kind is warp-uniform, so this is a predicated if-chain.  The
// staged-table form (OK_BUCKET_S) indexes the plan's int64 pool at tab_off.
__device__ __forceinline__ int64_t apply_id_op(const DevOp& op, const int64_t* itab, int64_t tab_off, int64_t v) {
  const int kind = op.kind;
  if (kind == OK_SIGRID) return (int64_t)reduce_M(splitmix_H(op.hsalt ^ (uint64_t)v), op.M);  // R3
  if (kind == OK_CLAMP) {                                                                       // R6
    v = v < op.a ? op.a : v;
    return v > op.b ? op.b : v;
  }
  if (kind == OK_BUCKET_S) return upper_bound(itab + tab_off + op.a, op.m, v);  // R4
  if (kind == OK_BUCKET_I) return upper_bound(itab + op.a, op.m, v);
  return map_lookup(itab, op.a, op.m, op.b, (int)op.M, (int64_t)op.hsalt, v);  // R8
}

__device__ __forceinline__ int64_t apply_id_ops(const DevOp* ops, const int64_t* itab, int64_t tab_off, int64_t v,
                                                int o0, int o1) {
  for (int o = o0; o < o1; ++o) v = apply_id_op(ops[o], itab, tab_off, v);
  return v;
}

// Register-resident pipeline of up to kPipe id ops (loaded once per tile;
// the ops are warp-uniform): per element the op itself plus a uniform branch.
constexpr int kPipe = 3;
struct Pipe {
  int n;
  int km[kPipe];  // kind | m << 8
  int64_t p0[kPipe], p1[kPipe];
};

__device__ __forceinline__ bool pipe_ok(const DevOp* ops, int o0, int o1) {
  if (o1 - o0 > kPipe) return false;
  for (int o = o0; o < o1; ++o)
    if (ops[o].kind == OK_MAPID && ops[o].M) return false;
  return true;
}

__device__ __forceinline__ void load_pipe(Pipe& pp, const DevOp* ops, int o0, int o1, int64_t tab_off) {
  pp.n = o1 - o0;
#pragma unroll
  for (int k = 0; k < kPipe; ++k) {
    pp.km[k] = -1;
    pp.p0[k] = pp.p1[k] = 0;
    if (k < pp.n) {
      const DevOp& op = ops[o0 + k];
      pp.km[k] = op.kind | (op.m << 8);
      if (op.kind == OK_SIGRID) {
        pp.p0[k] = (int64_t)op.hsalt;
        pp.p1[k] = op.M;
      } else {
        pp.p0[k] = op.kind == OK_BUCKET_S ? tab_off + op.a : op.a;
        pp.p1[k] = op.b;
      }
    }
  }
}

__device__ __forceinline__ int64_t run_pipe(const Pipe& pp, const int64_t* itab, int64_t v, int k0) {
#pragma unroll
  for (int k = 0; k < kPipe; ++k) {
    if (k >= k0 && k < pp.n) {
      const int kind = pp.km[k] & 0xff, m = pp.km[k] >> 8;
      if (kind == OK_SIGRID) {
        v = (int64_t)reduce_M(splitmix_H((uint64_t)pp.p0[k] ^ (uint64_t)v), pp.p1[k]);
      } else if (kind == OK_CLAMP) {
        v = v < pp.p0[k] ? pp.p0[k] : v;
        v = v > pp.p1[k] ? pp.p1[k] : v;
      } else if (kind == OK_MAPID) {
        v = map_lookup(itab, pp.p0[k], m, pp.p1[k], 0, 0, v);
      } else {  // OK_BUCKET_S / OK_BUCKET_I: p0 = absolute itab offset
        v = upper_bound(itab + pp.p0[k], m, v);
      }
    }
  }
  return v;
}

// Canonical pipeline (rap_internal.h): the stages present in MASK, in the
// fixed order Clamp -> MapId -> SigridHash -> Bucketize; `active` selects the
// stages of this element (all for a valid row, null_mask for a filled row).
template <int MASK>
__device__ __forceinline__ int64_t canon_apply(const Canon& q, const int64_t* itab, int64_t v, int active) {
  if ((MASK & CB_CLAMP) && (active & CB_CLAMP)) {  // R6
    v = v < q.lo ? q.lo : v;
    v = v > q.hi ? q.hi : v;
  }
  if ((MASK & CB_MAPID) && (active & CB_MAPID)) v = map_lookup(itab, q.map_a, q.map_m, q.map_def, 0, 0, v);  // R8
  if ((MASK & CB_SIGRID) && (active & CB_SIGRID))
    v = (int64_t)reduce_M(splitmix_H(q.hs ^ (uint64_t)v), q.M);                    // R3
  if ((MASK & CB_BUCKET) && (active & CB_BUCKET)) v = upper_bound(itab + q.bk_a, q.bk_m, v);  // R4
  return v;
}

// Calls body.template operator()<MASK>() for the runtime mask (16 cases).
#define RAP_CANON_DISPATCH(mask, CALL)   \
  switch ((mask) & 15) {                 \
    case 0: CALL(0); break;              \
    case 1: CALL(1); break;              \
    case 2: CALL(2); break;              \
    case 3: CALL(3); break;              \
    case 4: CALL(4); break;              \
    case 5: CALL(5); break;              \
    case 6: CALL(6); break;              \
    case 7: CALL(7); break;              \
    case 8: CALL(8); break;              \
    case 9: CALL(9); break;              \
    case 10: CALL(10); break;            \
    case 11: CALL(11); break;            \
    case 12: CALL(12); break;            \
    case 13: CALL(13); break;            \
    case 14: CALL(14); break;            \
    default: CALL(15); break;            \
  }

// Dense ops (R10-R12) in f32.
__device__ __forceinline__ float apply_dense_ops(const DevOp* ops, float x, int o0, int o1) {
  for (int o = o0; o < o1; ++o) {
    const DevOp& op = ops[o];
    if (op.kind == OK_FILL_F) {
      if (isnan(x)) x = op.f0;
    } else if (op.kind == OK_LOGIT) {
      const float z = x < op.f0 ? op.f0 : (x > op.f1 ? op.f1 : x);
      x = logf(__fdiv_rn(z, __fsub_rn(1.0f, z)));
    } else {  // OK_BOXCOX
      const float lam = op.f0;
      if (lam == 0.0f) {
        x = logf(x);
      } else {
        const float u = __fmul_rn(lam, logf(x));
        x = __fdiv_rn(expm1f(u), lam);
      }
    }
  }
  return x;
}

// Raw dense value from global memory with the R14 null rule (null -> NaN).
template <class P>
__device__ __forceinline__ float dense_raw(const P& p, int col, int64_t row) {
  const uint32_t* bm = p.dvalid[col];
  const uint32_t w = bm == nullptr ? 0xffffffffu : __ldg(bm + (row >> 5));
  const float x = __ldg(p.dense[col] + row);
  return ((w >> (row & 31)) & 1u) ? x : __int_as_float(0x7fc00000);
}

// ----------------------------------------------------------------------------
// Id-list sources.  For one row: the output length of a chain and the first
// child index (start >= 0), -1 for a filled null row (R10), -2 for a dense
// bucket (computed from the dense column).

struct RowIn {  // raw row data of one SRC_SPARSE source
  int32_t a, b;
  uint32_t w;  // validity word of the row's 32-row group
};

template <class P>
__device__ __forceinline__ RowIn load_row(const P& p, const Chain& ch, int64_t row, bool in) {
  RowIn r{0, 0, 0u};
  if (in && ch.src_kind == SRC_SPARSE) {
    const int32_t* off = p.off[ch.src];
    const uint32_t* bm = p.svalid[ch.src];
    r.a = __ldg(off + row);
    r.b = __ldg(off + row + 1);
    r.w = bm == nullptr ? 0xffffffffu : __ldg(bm + (row >> 5));
  }
  return r;
}

__device__ __forceinline__ int32_t row_len(const Chain& ch, const RowIn& r, int lane, bool in, int32_t* start) {
  if (!in) {
    *start = -1;
    return 0;
  }
  if (ch.src_kind != SRC_SPARSE) {
    *start = -2;  // SRC_DENSE_BUCKET: a length-1 list (R4)
    return (int32_t)min((int64_t)1, ch.xcap);
  }
  if ((r.w >> lane) & 1u) {
    *start = r.a;
    return (int32_t)min((int64_t)max(r.b - r.a, 0), ch.xcap);  // R5 FirstX as a cap
  }
  *start = -1;
  return ch.has_fill ? (int32_t)min((int64_t)1, ch.null_xcap) : 0;  // R10 / R14
}

// Element j of a source list (generic interpreter path).
template <class P>
__device__ __forceinline__ int64_t src_value(const P& p, const DevOp* ops, int64_t tab_off, const Chain& ch,
                                             int32_t start, int64_t row, int32_t j) {
  if (start >= 0) return apply_id_ops(ops, p.c.itab, tab_off, __ldg(p.val[ch.src] + start + j), ch.op_begin, ch.op_end);
  if (start == -1) return apply_id_ops(ops, p.c.itab, tab_off, ch.fill, ch.null_op_begin, ch.op_end);
  const float x = apply_dense_ops(ops, dense_raw(p, ch.src, row), ch.dop_begin, ch.dop_end);
  return apply_id_ops(ops, p.c.itab, tab_off, upper_bound(p.c.ftab + ch.btab, ch.bm, x), ch.op_begin, ch.op_end);
}

__device__ __forceinline__ const DevOp* prog_ops(const SProg& pg, const DevOp* gops) {
  return pg.global_ops ? gops : pg.ops;
}

// NGram window j (R7): h = H(salt); h = H(h ^ c[j+q]) for q < n; then the
// chain's post ops on reduce(h, M).  st[c * stride] / sl[c * stride]:
// per-source start / length of the row.
template <class P>
__device__ __noinline__ int64_t ngram_window(const P& p, const SProg& pg, const DevOp* ops, const int32_t* st,
                                             const int32_t* sl, int stride, int64_t row, int32_t j) {
  const int n = pg.ng.n;
  uint64_t h = pg.ng.hsalt;
  int c = 0;
  int32_t pos = j;
  for (int q = 0; q < n; ++q) {
    while (pos >= sl[c * stride]) {
      pos -= sl[c * stride];
      ++c;
    }
    const int64_t e = src_value(p, ops, pg.tab_off, pg.src[c], st[c * stride], row, pos);
    h = splitmix_H(h ^ (uint64_t)e);
    ++pos;
  }
  return apply_id_ops(ops, p.c.itab, pg.tab_off, (int64_t)reduce_M(h, pg.ng.M), pg.ch.op_begin, pg.ch.op_end);
}

__device__ __forceinline__ int warp_incl_scan(int v, int lane) {
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, v, d);
    if (lane >= d) v += y;
  }
  return v;
}

// ----------------------------------------------------------------------------
// Single-pass jagged scan (R17) over the feature-major sparse tile sequence:
// decoupled look-back.  Tile t publishes its length total (AGG) as soon as it
// is known, and later resolves its exclusive prefix by summing its
// predecessors' words, 32 per round trip, back to the nearest inclusive
// prefix (PREF), which it then publishes for itself.  Words carry the
// launch epoch, so they never need clearing between launches.
struct TileRef {
  unsigned long long* status;
  long long t;
  unsigned long long tag;  // epoch << kEpochShift
};

__device__ __forceinline__ void publish_agg(const TileRef& tr, long long T, int lane) {
  if (lane == 0) st_relaxed(tr.status + tr.t, tr.tag | (kFlagAgg << kFlagShift) | (unsigned long long)T);
}

__device__ __forceinline__ long long tile_lookback(const TileRef& tr, long long T, int lane) {
  const unsigned long long epoch = tr.tag >> kEpochShift;
  long long excl = 0;
  long long top = tr.t - 1;
  while (top >= 0) {
    const long long idx = top - lane;
    unsigned long long w = 0;
    unsigned pm, take;
    while (true) {
      int fl = (int)kFlagPrefix;  // before tile 0: an inclusive prefix of 0
      w = 0;
      if (idx >= 0) {
        w = ld_relaxed(tr.status + idx);
        fl = (w >> kEpochShift) == epoch ? (int)((w >> kFlagShift) & 3ull) : 0;
      }
      pm = __ballot_sync(0xffffffffu, fl == (int)kFlagPrefix);
      const unsigned zm = __ballot_sync(0xffffffffu, fl == 0);
      take = pm ? ((pm & (0u - pm)) << 1) - 1u : 0xffffffffu;  // lanes up to the nearest prefix
      if ((zm & take) == 0) break;
      __nanosleep(32);
    }
    excl += warp_sum64(((take >> lane) & 1u) ? (long long)(w & kValueMask) : 0ll);
    if (pm) break;
    top -= 32;
  }
  if (lane == 0) st_relaxed(tr.status + tr.t, tr.tag | (kFlagPrefix << kFlagShift) | (unsigned long long)(excl + T));
  return excl;
}

// ----------------------------------------------------------------------------
// Sparse tiles with 4 consecutive rows per lane (rows r0 + 4*lane + k): one
// 16-byte offsets load, one validity word, 16-byte length / offset stores.

// Per-feature state a warp keeps in registers across its tiles.
struct FeatCtx {
  int f, kind, src, has_fill, canon, mask;
  int64_t xcap, null_xcap, fill;
  Canon q;
};

template <class P>
__device__ __forceinline__ void load_ctx(const P& p, int f, FeatCtx& x) {
  const SProg& pg = p.c.sprogs[f];
  x.f = f;
  x.kind = pg.ch.src_kind;
  x.src = pg.ch.src;
  x.has_fill = pg.ch.has_fill;
  x.xcap = pg.ch.xcap;
  x.null_xcap = pg.ch.null_xcap;
  x.fill = pg.ch.fill;
  x.q = pg.cn;
  x.canon = x.q.ok && x.kind == SRC_SPARSE;
  x.mask = x.q.mask;
}

// Arrow offsets of rows r0+4*lane .. +4 and the validity word of those rows.
struct Quad {
  int32_t a[5];
  uint32_t w;
};

__device__ __forceinline__ Quad load_quad(const int32_t* off, const uint32_t* bm, int64_t r0, int lane, int64_t B,
                                          bool aligned) {
  Quad q;
  const int64_t row = r0 + 4 * lane;
  if (aligned && row + 4 <= B) {
    const int4 v = __ldg(reinterpret_cast<const int4*>(off + row));
    q.a[0] = v.x;
    q.a[1] = v.y;
    q.a[2] = v.z;
    q.a[3] = v.w;
    q.a[4] = __ldg(off + row + 4);
  } else {
#pragma unroll
    for (int k = 0; k < 5; ++k) q.a[k] = row + k <= B ? __ldg(off + row + k) : 0;
  }
  q.w = (bm != nullptr && row < B) ? __ldg(bm + (row >> 5)) : 0xffffffffu;
  return q;
}

// Output length of row k of the quad (R5 FirstX cap, R10 fill, R14 null).
__device__ __forceinline__ int32_t quad_len(const Quad& q, int k, int lane, int64_t row, int64_t B, int64_t xcap,
                                            int has_fill, int64_t null_xcap) {
  if (row >= B) return 0;
  if ((q.w >> ((4 * lane + k) & 31)) & 1u) return (int32_t)min((int64_t)max(q.a[k + 1] - q.a[k], 0), xcap);
  return has_fill ? (int32_t)min((int64_t)1, null_xcap) : 0;
}

__device__ __forceinline__ bool quad_valid(const Quad& q, int k, int lane) {
  return (q.w >> ((4 * lane + k) & 31)) & 1u;
}

// ----------------------------------------------------------------------------
// Phase 3: offsets and ids of sparse tile (f, rt), whose first output id goes
// to values[base].
template <class P>
__device__ __noinline__ void value_group_general(const P& p, int f, int64_t row0, int lane, int32_t mylen,
                                                 int32_t myst, int32_t lx, long long gbase);
template <class P>
__device__ __noinline__ void value_tile_ngram(const P& p, int f, int64_t rt, int lane, const TileRef& tr,
                                              int32_t* scr);

// Lengths (int4) and offsets (2 x longlong2) of the lane's 4 rows.
__device__ __forceinline__ void store_quad(int32_t* lp, int64_t* op, int64_t row, int64_t B, const int32_t* l,
                                           long long lb, const int32_t* e) {
  if (row + 4 <= B && (reinterpret_cast<uintptr_t>(lp) & 15) == 0 && (reinterpret_cast<uintptr_t>(op) & 15) == 0) {
    *reinterpret_cast<int4*>(lp) = make_int4(l[0], l[1], l[2], l[3]);
    reinterpret_cast<longlong2*>(op)[0] = make_longlong2(lb + e[0], lb + e[1]);
    reinterpret_cast<longlong2*>(op)[1] = make_longlong2(lb + e[2], lb + e[3]);
  } else {
#pragma unroll
    for (int k = 0; k < 4; ++k)
      if (row + k < B) {
        lp[k] = l[k];
        op[k] = lb + e[k];
      }
  }
}

// Specialised tile of a canonical SRC_SPARSE chain (mask MASK); the lane
// owns rows r0 + 4*lane + k, so its output ids are contiguous.
template <int MASK, class P>
__device__ __noinline__ void value_tile_canon(const P& p, const FeatCtx& fc, int64_t rt, int lane, const TileRef& tr) {
  const Canon& q = fc.q;
  const int f = fc.f;
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rt * kTileRows;
  const int64_t row = r0 + 4 * lane;
  int64_t* values = p.c.values;
  const long long cap = p.c.values_cap;
  const int64_t* itab = p.c.itab;
  const int32_t* off = p.off[fc.src];
  const int64_t* val = p.val[fc.src];
  const Quad qd = load_quad(off, p.svalid[fc.src], r0, lane, B, (reinterpret_cast<uintptr_t>(off) & 15) == 0);
  int32_t l[4], e[4];
  int tot = 0;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    l[k] = quad_len(qd, k, lane, row + k, B, fc.xcap, fc.has_fill, fc.null_xcap);
    e[k] = tot;
    tot += l[k];
  }
  const int incl = warp_incl_scan(tot, lane);
  const int L = incl - tot;  // lane exclusive prefix within the tile
  const int T = __shfl_sync(0xffffffffu, incl, 31);
  publish_agg(tr, T, lane);
  const bool last = f == p.c.n_sparse_out - 1 && rt == p.c.tiles_per_feature - 1;
  int32_t* lp = p.c.lengths + (int64_t)f * B + row;
  int64_t* op = p.c.offsets + (int64_t)f * B + row;
  if (__all_sync(0xffffffffu, l[0] <= 1 && l[1] <= 1 && l[2] <= 1 && l[3] <= 1)) {
    // at most one id per row: the ids are computed before the base is known
    int64_t v[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) v[k] = (l[k] == 1 && quad_valid(qd, k, lane)) ? __ldg(val + qd.a[k]) : fc.fill;
#pragma unroll
    for (int k = 0; k < 4; ++k)
      if (l[k] == 1) v[k] = canon_apply<MASK>(q, itab, v[k], quad_valid(qd, k, lane) ? 15 : q.null_mask);
    const long long base = tile_lookback(tr, T, lane);
    const long long lb = base + L;
    store_quad(lp, op, row, B, l, lb, e);
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const long long pos = lb + e[k];
      if (l[k] == 1 && pos < cap) values[pos] = v[k];
    }
    if (last && lane == 31) {
      p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + T;  // total, R17
      if (base + T > cap) atomicExch(p.c.err, 1);
    }
    return;
  }
  const long long base = tile_lookback(tr, T, lane);
  store_quad(lp, op, row, B, l, base + L, e);
  if (last && lane == 31) {
    p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + T;
    if (base + T > cap) atomicExch(p.c.err, 1);
  }
  // multi-id rows: elements in output order; owning lane by a 5-step shuffle
  // search over the lane prefixes, then the row within the lane
  const int mylex = L;
  for (int eb = 0; eb < T; eb += 32) {
    const int ee = eb + lane;
    int r = 0;
#pragma unroll
    for (int step = 16; step >= 1; step >>= 1) {
      const int c = __shfl_sync(0xffffffffu, mylex, r + step);
      if (c <= ee) r += step;
    }
    const int in_lane = ee - __shfl_sync(0xffffffffu, mylex, r);
    const int e1 = __shfl_sync(0xffffffffu, e[1], r), e2 = __shfl_sync(0xffffffffu, e[2], r),
              e3 = __shfl_sync(0xffffffffu, e[3], r);
    const int k = in_lane >= e3 ? 3 : (in_lane >= e2 ? 2 : (in_lane >= e1 ? 1 : 0));
    const int ek = k == 3 ? e3 : (k == 2 ? e2 : (k == 1 ? e1 : 0));
    const int32_t a0 = __shfl_sync(0xffffffffu, qd.a[0], r), a1 = __shfl_sync(0xffffffffu, qd.a[1], r),
                  a2 = __shfl_sync(0xffffffffu, qd.a[2], r), a3 = __shfl_sync(0xffffffffu, qd.a[3], r);
    const uint32_t wr = __shfl_sync(0xffffffffu, qd.w, r);
    const int32_t ak = k == 3 ? a3 : (k == 2 ? a2 : (k == 1 ? a1 : a0));
    const bool vk = (wr >> ((4 * r + k) & 31)) & 1u;
    if (ee < T) {
      const int64_t x = vk ? __ldg(val + ak + (in_lane - ek)) : fc.fill;
      const int64_t v = canon_apply<MASK>(q, itab, x, vk ? 15 : q.null_mask);
      const long long pos = base + ee;
      if (pos < cap) values[pos] = v;
    }
  }
}

// Tile of any other SRC_SPARSE / SRC_DENSE_BUCKET chain (op interpreter).
template <class P>
__device__ __noinline__ void value_tile_generic(const P& p, int f, int64_t rt, int lane, const TileRef& tr) {
  const SProg& pg = p.c.sprogs[f];
  const DevOp* ops = prog_ops(pg, p.c.ops);
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rt * kTileRows;
  int64_t* offsets = p.c.offsets + (int64_t)f * B;
  int32_t* lengths = p.c.lengths + (int64_t)f * B;
  int64_t* values = p.c.values;
  const long long cap = p.c.values_cap;
  const int64_t* itab = p.c.itab;
  const Chain ch = pg.ch;
  // all row loads of the tile first (kGroups independent requests per lane)
  RowIn in[kGroups];
#pragma unroll
  for (int g = 0; g < kGroups; ++g) {
    const int64_t row = r0 + 32 * g + lane;
    in[g] = load_row(p, ch, row, row < B);
  }
  int32_t len[kGroups], st[kGroups], lex[kGroups], gb[kGroups];
  bool all1 = true;
  int run = 0;  // tile-relative
#pragma unroll
  for (int g = 0; g < kGroups; ++g) {
    const int64_t row = r0 + 32 * g + lane;
    len[g] = row_len(ch, in[g], lane, row < B, &st[g]);
    all1 &= len[g] <= 1;
    const int incl = warp_incl_scan(len[g], lane);
    lex[g] = incl - len[g];
    gb[g] = run;
    run += __shfl_sync(0xffffffffu, incl, 31);
  }
  publish_agg(tr, run, lane);
  const bool use_pipe = ch.src_kind == SRC_SPARSE && pipe_ok(ops, ch.op_begin, ch.op_end);
  Pipe pipe;
  if (use_pipe) load_pipe(pipe, ops, ch.op_begin, ch.op_end, pg.tab_off);
  const int null_k0 = ch.null_op_begin - ch.op_begin;
  all1 = __all_sync(0xffffffffu, all1);
  int64_t v1[kGroups];
  if (all1) {
    // one id per row at most: ids computed before the base is known
#pragma unroll
    for (int g = 0; g < kGroups; ++g)
      v1[g] = (len[g] == 1 && st[g] >= 0) ? __ldg(p.val[ch.src] + st[g]) : ch.fill;
#pragma unroll
    for (int g = 0; g < kGroups; ++g) {
      if (len[g] == 1) {
        const int64_t row = r0 + 32 * g + lane;
        v1[g] = use_pipe ? run_pipe(pipe, itab, v1[g], st[g] >= 0 ? 0 : null_k0)
                         : src_value(p, ops, pg.tab_off, ch, st[g], row, 0);
      }
    }
  }
  const long long base = tile_lookback(tr, run, lane);
#pragma unroll
  for (int g = 0; g < kGroups; ++g) {
    const int64_t row = r0 + 32 * g + lane;
    if (row < B) {
      lengths[row] = len[g];
      offsets[row] = base + gb[g] + lex[g];
    }
  }
  if (f == p.c.n_sparse_out - 1 && rt == p.c.tiles_per_feature - 1 && lane == 0) {
    p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + run;  // total, R17
    if (base + run > cap) atomicExch(p.c.err, 1);
  }
  if (all1) {
#pragma unroll
    for (int g = 0; g < kGroups; ++g) {
      const long long pos = base + gb[g] + lex[g];
      if (len[g] == 1 && pos < cap) values[pos] = v1[g];
    }
    return;
  }
  // general (multi-id rows): elements in output order, per row group
#pragma unroll 1
  for (int g = 0; g < kGroups; ++g)
    value_group_general(p, f, r0 + 32 * g, lane, len[g], st[g], lex[g], base + gb[g]);
}

template <class P>
__device__ __forceinline__ void value_tile(const P& p, const FeatCtx& fc, int64_t rt, int lane, const TileRef& tr,
                                           int32_t* scr) {
  if (fc.canon) {
#define RAP_VT_CALL(M) value_tile_canon<M>(p, fc, rt, lane, tr)
    RAP_CANON_DISPATCH(fc.mask, RAP_VT_CALL)
#undef RAP_VT_CALL
  } else if (fc.kind == SRC_NGRAM) {
    value_tile_ngram(p, fc.f, rt, lane, tr, scr);
  } else {
    value_tile_generic(p, fc.f, rt, lane, tr);
  }
}

// Ids of one 32-row group with multi-id rows: elements in output order, the
// owning row found by a 5-step shuffle search over the lanes' exclusive prefixes.
template <class P>
__device__ __noinline__ void value_group_general(const P& p, int f, int64_t row0, int lane, int32_t mylen,
                                                 int32_t myst, int32_t lx, long long gbase) {
  const SProg& pg = p.c.sprogs[f];
  const DevOp* ops = prog_ops(pg, p.c.ops);
  const Chain& ch = pg.ch;
  const long long cap = p.c.values_cap;
  const bool use_pipe = ch.src_kind == SRC_SPARSE && pipe_ok(ops, ch.op_begin, ch.op_end);
  Pipe pipe;
  if (use_pipe) load_pipe(pipe, ops, ch.op_begin, ch.op_end, pg.tab_off);
  const int null_k0 = ch.null_op_begin - ch.op_begin;
  const int T = __shfl_sync(0xffffffffu, lx + mylen, 31);
  const int mylex = (row0 + lane < p.c.n_rows) ? lx : INT_MAX;
  for (int eb = 0; eb < T; eb += 32) {
    const int e = eb + lane;
    int r = 0;
#pragma unroll
    for (int step = 16; step >= 1; step >>= 1) {
      const int c = __shfl_sync(0xffffffffu, mylex, r + step);
      if (c <= e) r += step;
    }
    const int lex_r = __shfl_sync(0xffffffffu, mylex, r);
    const int32_t st_r = __shfl_sync(0xffffffffu, myst, r);
    if (e < T) {
      const int32_t j = e - lex_r;
      int64_t v;
      if (use_pipe) {
        const int64_t x = st_r >= 0 ? __ldg(p.val[ch.src] + st_r + j) : ch.fill;
        v = run_pipe(pipe, p.c.itab, x, st_r >= 0 ? 0 : null_k0);
      } else {
        v = src_value(p, ops, pg.tab_off, ch, st_r, row0 + r, j);
      }
      const long long pos = gbase + e;
      if (pos < cap) p.c.values[pos] = v;
    }
  }
}

// NGram feature tile (R7): per row the k source lists, windows over their
// concatenation.
template <class P>
__device__ __noinline__ void value_tile_ngram(const P& p, int f, int64_t rt, int lane, const TileRef& tr,
                                              int32_t* scr) {
  const SProg& pg = p.c.sprogs[f];
  const DevOp* ops = prog_ops(pg, p.c.ops);
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rt * kTileRows;
  int64_t* offsets = p.c.offsets + (int64_t)f * B;
  int32_t* lengths = p.c.lengths + (int64_t)f * B;
  int64_t* values = p.c.values;
  const long long cap = p.c.values_cap;
  // pass 1: the tile's output length total (quad layout: 4 rows per lane,
  // every source's offsets requested before any is used), published at once
  long long base;
  {
    int32_t tot4[4] = {0, 0, 0, 0};
#pragma unroll 1
    for (int c0 = 0; c0 < pg.ng.k; c0 += 4) {  // 4 sources' offsets in flight at a time
      Quad qs[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int c = c0 + j;
        if (c < pg.ng.k && pg.src[c].src_kind == SRC_SPARSE) {
          const int32_t* off = p.off[pg.src[c].src];
          qs[j] = load_quad(off, p.svalid[pg.src[c].src], r0, lane, B, (reinterpret_cast<uintptr_t>(off) & 15) == 0);
        }
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int c = c0 + j;
        if (c < pg.ng.k) {
          const Chain& sc = pg.src[c];
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const int64_t row = r0 + 4 * lane + q;
            if (sc.src_kind == SRC_SPARSE)
              tot4[q] += quad_len(qs[j], q, lane, row, B, sc.xcap, sc.has_fill, sc.null_xcap);
            else
              tot4[q] += row < B ? (int32_t)min((int64_t)1, sc.xcap) : 0;
          }
        }
      }
    }
    int sum = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q)
      if (r0 + 4 * lane + q < B) sum += (int32_t)min((int64_t)max(tot4[q] - pg.ng.n + 1, 0), pg.ch.xcap);
    const long long T = warp_sum64(sum);
    publish_agg(tr, T, lane);
    base = tile_lookback(tr, T, lane);
  }

  // NGram feature (R7): per row the k source lists, windows over their
  // concatenation.  Per-source (start, length) of the warp's 32 rows live in
  // warp-private shared memory: scr[c*32 + lane] / scr[(kMaxNgramK + c)*32 + lane].
  const int k = pg.ng.k, n = pg.ng.n;
  const int64_t xcap = pg.ch.xcap;
  int32_t* st_s = scr;
  int32_t* sl_s = scr + kMaxNgramK * 32;
  int64_t* ev_s = reinterpret_cast<int64_t*>(scr + 2 * kMaxNgramK * 32);  // [c][lane] element ids
  const int64_t* itab = p.c.itab;
  // canonical fast path: every source (and the post-hash ops) canonical
  bool canon_all = pg.cn.ok;
  for (int c = 0; c < k; ++c) canon_all &= pg.src_cn[c].ok != 0;
  long long run = base;
#pragma unroll 1
  for (int g = 0; g < kGroups; ++g) {
    const int64_t row = r0 + 32 * g + lane;
    const bool inr = row < B;
    RowIn in[kMaxNgramK];
#pragma unroll
    for (int c = 0; c < kMaxNgramK; ++c)
      if (c < k) in[c] = load_row(p, pg.src[c], row, inr);
    int tot = 0, slmax = 0;
#pragma unroll
    for (int c = 0; c < kMaxNgramK; ++c) {
      if (c < k) {
        int32_t st;
        const int32_t sl = row_len(pg.src[c], in[c], lane, inr, &st);
        st_s[c * 32 + lane] = st;
        sl_s[c * 32 + lane] = sl;
        tot += sl;
        slmax = max(slmax, sl);
        if (canon_all) ev_s[c * 32 + lane] = (sl >= 1 && st >= 0) ? __ldg(p.val[pg.src[c].src] + st) : pg.src[c].fill;
      }
    }
    __syncwarp();
    const int32_t len = inr ? (int32_t)min((int64_t)max(tot - n + 1, 0), xcap) : 0;
    const int incl = warp_incl_scan(len, lane);
    const int lx = incl - len;
    const int T = __shfl_sync(0xffffffffu, incl, 31);
    if (inr) {
      lengths[row] = len;
      offsets[row] = run + lx;
    }
    if (canon_all && __all_sync(0xffffffffu, slmax <= 1)) {
      // single-id sources: run each source's canonical pipeline once per row,
      // then hash the windows from the staged ids
      unsigned present = 0;
      for (int c = 0; c < k; ++c) {
        const Canon qc = pg.src_cn[c];
        const int sl = sl_s[c * 32 + lane];
        if (sl == 1) {
          present |= 1u << c;
          const int act = st_s[c * 32 + lane] >= 0 ? 15 : qc.null_mask;
          int64_t x = ev_s[c * 32 + lane];
#define RAP_NG_CALL(M) x = canon_apply<M>(qc, itab, x, act)
          RAP_CANON_DISPATCH(qc.mask, RAP_NG_CALL)
#undef RAP_NG_CALL
          ev_s[c * 32 + lane] = x;
        }
      }
      const Canon qp = pg.cn;
      for (int j = 0; j < len; ++j) {
        uint64_t h = pg.ng.hsalt;  // R7: h = H(salt); h = H(h ^ c[j+q])
        int seen = 0, q = 0;
        for (int c = 0; c < k && q < n; ++c) {
          if ((present >> c) & 1u) {
            if (seen >= j) {
              h = splitmix_H(h ^ (uint64_t)ev_s[c * 32 + lane]);
              ++q;
            }
            ++seen;
          }
        }
        int64_t v = (int64_t)reduce_M(h, pg.ng.M);
#define RAP_NP_CALL(M) v = canon_apply<M>(qp, itab, v, 15)
        RAP_CANON_DISPATCH(qp.mask, RAP_NP_CALL)
#undef RAP_NP_CALL
        const long long pos = run + lx + j;
        if (pos < cap) values[pos] = v;
      }
    } else if (__all_sync(0xffffffffu, len <= 1)) {
      if (len == 1) {
        const long long pos = run + lx;
        const int64_t v = ngram_window(p, pg, ops, st_s + lane, sl_s + lane, 32, row, 0);
        if (pos < cap) values[pos] = v;
      }
    } else {
      const int mylex = inr ? lx : INT_MAX;
      for (int eb = 0; eb < T; eb += 32) {
        const int e = eb + lane;
        int r = 0;
#pragma unroll
        for (int step = 16; step >= 1; step >>= 1) {
          const int c = __shfl_sync(0xffffffffu, mylex, r + step);
          if (c <= e) r += step;
        }
        const int lex_r = __shfl_sync(0xffffffffu, mylex, r);
        if (e < T) {
          const int64_t v = ngram_window(p, pg, ops, st_s + r, sl_s + r, 32, r0 + 32 * g + r, e - lex_r);
          const long long pos = run + e;
          if (pos < cap) values[pos] = v;
        }
      }
    }
    __syncwarp();
    run += T;
  }
  if (f == p.c.n_sparse_out - 1 && rt == p.c.tiles_per_feature - 1 && lane == 0) {
    p.c.offsets[(int64_t)p.c.n_sparse_out * B] = run;
    if (run > cap) atomicExch(p.c.err, 1);
  }
}

// ----------------------------------------------------------------------------
// Dense block: kDenseBlockRows rows of one column group -> row-major tile via
// smem (a2).  Inputs staged with bulk copies on the CTA mbarrier.
struct CtaState {
  uint64_t bar;
  long long ticket;
  int staged, phase;
};

constexpr int kDProgBytes = align_up((int)sizeof(DProg), 16);

__host__ __device__ constexpr int dense_in_bytes() { return 16 * kDenseBlockRows * 4 + 16 * 8 * 4; }

// OneHot over a generic id list (sparse list, NGram windows): set the columns
// of the ids in [k0, k0+width) in the row's tile slice (R9).
template <class P>
__device__ __noinline__ void onehot_generic(const P& p, const DUnit& un, int64_t row, float* trow) {
  const SProg& og = p.c.oprogs[un.prog];
  const DevOp* gops = prog_ops(og, p.c.ops);
  const int ln = (int)(row & 31);
  int32_t st[kMaxNgramK], sl[kMaxNgramK];
  if (og.ch.src_kind != SRC_NGRAM) {
    const RowIn ri = load_row(p, og.ch, row, true);
    const int32_t L = row_len(og.ch, ri, ln, true, &st[0]);
    for (int32_t j = 0; j < L; ++j) {
      const int64_t d = src_value(p, gops, og.tab_off, og.ch, st[0], row, j) - un.k0;
      if (d >= 0 && d < un.width) trow[un.col + (int)d] = 1.0f;
    }
    return;
  }
  int tot = 0;
  for (int c = 0; c < og.ng.k; ++c) {
    const RowIn ri = load_row(p, og.src[c], row, true);
    sl[c] = row_len(og.src[c], ri, ln, true, &st[c]);
    tot += sl[c];
  }
  const int32_t L = (int32_t)min((int64_t)max(tot - og.ng.n + 1, 0), og.ch.xcap);
  for (int32_t j = 0; j < L; ++j) {
    const int64_t d = ngram_window(p, og, gops, st, sl, 1, row, j) - un.k0;
    if (d >= 0 && d < un.width) trow[un.col + (int)d] = 1.0f;
  }
}

template <class P>
__device__ void dense_block(const P& p, int gi, int64_t rb, unsigned char* smem, CtaState& cs) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  DProg* dp = reinterpret_cast<DProg*>(smem);
  float* din = reinterpret_cast<float*>(smem + kDProgBytes);  // [16][kDenseBlockRows]
  uint32_t* dbm = reinterpret_cast<uint32_t*>(smem + kDProgBytes + 16 * kDenseBlockRows * 4);  // [16][8]
  float* tile = reinterpret_cast<float*>(smem + kDProgBytes + dense_in_bytes());
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rb * kDenseBlockRows;
  const int nr = (int)min((int64_t)kDenseBlockRows, B - r0);
  const int nw = (nr + 31) >> 5;
  if (warp == 0) {
    const DProg* g = p.c.dprogs + gi;
    const int nu = __ldg(&g->n_units), no = __ldg(&g->n_ops), nf = __ldg(&g->n_ftab), nc = __ldg(&g->n_cols);
    const int col = lane < nc ? __ldg(&g->cols[lane]) : 0;
    const bool aligned = lane >= nc || ((reinterpret_cast<uintptr_t>(p.dense[col] + r0) & 15) == 0 &&
                                        (p.dvalid[col] == nullptr ||
                                         (reinterpret_cast<uintptr_t>(p.dvalid[col] + (r0 >> 5)) & 15) == 0));
    const bool stage = __all_sync(0xffffffffu, aligned) && (nr & 3) == 0 && nc <= 16;
    if (stage) {
      const uint32_t bytes_v = (uint32_t)nr * 4, bytes_b = (uint32_t)align_up(nw * 4, 16);
      uint32_t total = 0;
      if (lane < nc) total = bytes_v + (p.dvalid[col] ? bytes_b : 0);
#pragma unroll
      for (int d = 16; d >= 1; d >>= 1) total += __shfl_xor_sync(0xffffffffu, total, d);
      if (lane == 0) {
        fence_proxy_async();
        mbar_arrive_expect(&cs.bar, total);
      }
      __syncwarp();
      if (lane < nc) {
        bulk_g2s(din + lane * kDenseBlockRows, p.dense[col] + r0, bytes_v, &cs.bar);
        if (p.dvalid[col]) bulk_g2s(dbm + lane * 8, p.dvalid[col] + (r0 >> 5), bytes_b, &cs.bar);
      }
    }
    if (lane == 0) cs.staged = stage ? 1 : 0;
    const int4* src = reinterpret_cast<const int4*>(g);
    int4* dst = reinterpret_cast<int4*>(dp);
    const int n_hdr = align_up((int)offsetof(DProg, units) + nu * (int)sizeof(DUnit), 16) >> 4;
    for (int k = lane; k < n_hdr; k += 32) dst[k] = __ldg(src + k);
    const int4* so = reinterpret_cast<const int4*>(g->ops);
    int4* d2 = reinterpret_cast<int4*>(dp->ops);
    for (int k = lane; k < (align_up(no * (int)sizeof(DevOp), 16) >> 4); k += 32) d2[k] = __ldg(so + k);
    const int4* sf = reinterpret_cast<const int4*>(g->ftab);
    int4* d3 = reinterpret_cast<int4*>(dp->ftab);
    for (int k = lane; k < (align_up(nf * 4, 16) >> 4); k += 32) d3[k] = __ldg(sf + k);
  }
  __syncthreads();
  const int W = dp->width;
  const int LD = W | 1;  // odd row pitch: conflict-free column writes
  if (dp->any_onehot)
    for (int i = tid; i < nr * LD; i += kThreads) tile[i] = 0.0f;
  const bool staged = cs.staged;
  if (staged) mbar_wait(&cs.bar, cs.phase);
  __syncthreads();
  const int nu = dp->n_units;
  // (row, unit) pairs over all threads, unit-major so a warp shares its unit
  for (int idx = tid; idx < nr * nu; idx += kThreads) {
    const int u = idx / nr, r = idx - u * nr;
    const int64_t row = r0 + r;
    const DUnit& un = dp->units[u];
    const DevOp* uops = un.gops ? p.c.ops : dp->ops;
    if (un.kind == U_ONEHOT_G) {  // generic list (R9), program from global memory
      onehot_generic(p, un, row, tile + r * LD);
      continue;
    }
    float x;
    if (staged) {
      const uint32_t w = p.dvalid[un.src_col] ? dbm[un.slot * 8 + (r >> 5)] : 0xffffffffu;
      x = ((w >> (r & 31)) & 1u) ? din[un.slot * kDenseBlockRows + r] : __int_as_float(0x7fc00000);
    } else {
      x = dense_raw(p, un.src_col, row);
    }
    x = apply_dense_ops(uops, x, un.op_begin, un.op_end);
    if (un.kind == U_DENSE) {
      tile[r * LD + un.col] = x;
    } else if (un.xcap > 0) {  // U_ONEHOT_DB
      const float* uft = un.gops ? p.c.ftab : dp->ftab;
      const int64_t bidx = un.gops ? upper_bound(uft + un.btab, un.bm, x) : upper_bound_s(uft + un.btab, un.bm, x);
      const int64_t id = apply_id_ops(uops, p.c.itab, 0, bidx, un.iop_begin, un.iop_end);
      const int64_t d = id - un.k0;
      if (d >= 0 && d < un.width) tile[r * LD + un.col + (int)d] = 1.0f;
    }
  }
  __syncthreads();
  float* out = p.c.dense_out + r0 * p.c.ld + dp->col0;
  const int64_t ld = p.c.ld;
  if (ld == W && LD == W) {
    const int n = nr * W;  // the block is one contiguous run
    if ((reinterpret_cast<uintptr_t>(out) & 15) == 0 && (n & 3) == 0) {
      float4* o4 = reinterpret_cast<float4*>(out);
      const float4* t4 = reinterpret_cast<const float4*>(tile);
      for (int i = tid; i < (n >> 2); i += kThreads) o4[i] = t4[i];
    } else {
      for (int i = tid; i < n; i += kThreads) out[i] = tile[i];
    }
  } else {
    for (int r = warp; r < nr; r += kWarps)
      for (int cc = lane; cc < W; cc += 32) out[r * ld + cc] = tile[r * LD + cc];
  }
  if (tid == 0 && staged) cs.phase ^= 1;
}

// ----------------------------------------------------------------------------
#ifndef RAP_MIN_CTAS
#define RAP_MIN_CTAS 4
#endif
template <int MD, int MS>
__global__ void __launch_bounds__(kThreads, RAP_MIN_CTAS) rap_fused_kernel(const __grid_constant__ KParams<MD, MS> p) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ CtaState cs;
  __shared__ long long s_item;
  __shared__ unsigned long long s_epoch;
  __shared__ int s_last;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    mbar_init(&cs.bar, 1);
    cs.phase = 0;
    s_epoch = ld_relaxed(p.c.sched + 1);
  }
  __syncthreads();
  trace_stamp(p.c, 0);
  const unsigned long long epoch = s_epoch;

  // (1) sparse tiles (warp units) from a global queue, in scan order
  {
    FeatCtx fc;
    fc.f = -1;
    int32_t* scr = reinterpret_cast<int32_t*>(smem) + warp * (4 * kMaxNgramK * 32);
    const int64_t S = p.c.n_sparse_tiles, T = p.c.tiles_per_feature;
    TileRef tr;
    tr.status = p.c.status;
    tr.tag = epoch << kEpochShift;
    while (true) {
      long long t = 0;
      if (lane == 0) t = (long long)atomicAdd(p.c.sched + 3, 1ull);
      t = __shfl_sync(0xffffffffu, t, 0);
      if (t >= S) break;
      const int f = (int)((uint64_t)t / (uint64_t)T);
      if (f != fc.f) load_ctx(p, f, fc);
      tr.t = t;
      value_tile(p, fc, (int64_t)t - (int64_t)f * T, lane, tr, scr);
    }
  }
  trace_stamp(p.c, 1);
  __syncthreads();

  // (2) dense blocks (CTA units) from a second global queue
  while (true) {
    if (tid == 0) s_item = (long long)atomicAdd(p.c.sched + 2, 1ull);
    __syncthreads();
    const long long d = s_item;
    __syncthreads();
    if (d >= p.c.n_dense_tiles) break;
    const uint32_t gi = (uint32_t)d % (uint32_t)p.c.n_groups;
    dense_block(p, (int)gi, (int64_t)((uint32_t)d / (uint32_t)p.c.n_groups), smem, cs);
    __syncthreads();
  }
  trace_stamp(p.c, 2);

  // The last CTA out resets the queue heads and advances the epoch of the
  // look-back words (clearing them when the 20-bit epoch wraps), so launch
  // parameters are identical from call to call (CUDA-graph replayable).
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    const unsigned long long prev = atomicAdd(p.c.sched, 1ull);
    s_last = (prev == (unsigned long long)gridDim.x - 1) ? 1 : 0;
    if (s_last) __threadfence();
  }
  __syncthreads();
  if (s_last) {
    const bool wrap = epoch >= kEpochMax;
    if (wrap)
      for (int64_t i = tid; i < p.c.n_sparse_tiles; i += kThreads) p.c.status[i] = 0ull;
    __syncthreads();
    if (tid == 0) {
      p.c.sched[0] = 0ull;
      p.c.sched[2] = 0ull;
      p.c.sched[3] = 0ull;
      p.c.sched[1] = wrap ? 1ull : epoch + 1ull;
      __threadfence();
    }
  }
}

template <int MD, int MS>
static int launch_t(const Common& c, const LaunchRaw& raw, int grid, int smem, cudaStream_t st) {
  static_assert(sizeof(KParams<MD, MS>) <= 32000, "kernel parameter block too large");
  static int configured_smem = -1;
  if (configured_smem < smem) {
    cudaError_t e = cudaFuncSetAttribute(rap_fused_kernel<MD, MS>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return (int)e;
    configured_smem = smem;
  }
  KParams<MD, MS> p;
  memset(&p, 0, sizeof(p));
  p.c = c;
  for (int i = 0; i < raw.n_dense; ++i) {
    p.dense[i] = raw.dense[i];
    p.dvalid[i] = raw.dvalid ? raw.dvalid[i] : nullptr;
  }
  for (int i = 0; i < raw.n_sparse; ++i) {
    p.off[i] = raw.off[i];
    p.val[i] = raw.val[i];
    p.svalid[i] = raw.svalid ? raw.svalid[i] : nullptr;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cfg.numAttrs = 0;
  cudaError_t e = cudaLaunchKernelEx(&cfg, rap_fused_kernel<MD, MS>, p);
  if (e != cudaSuccess) return (int)e;
  return (int)cudaGetLastError();
}

int launch_fused(const Common& c, const LaunchRaw& raw, int grid, int smem_bytes, void* stream) {
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (grid > kMaxCtas) return (int)cudaErrorInvalidValue;
  if (raw.n_dense <= 32 && raw.n_sparse <= 64) return launch_t<32, 64>(c, raw, grid, smem_bytes, st);
  if (raw.n_dense <= 128 && raw.n_sparse <= 1024) return launch_t<128, 1024>(c, raw, grid, smem_bytes, st);
  return (int)cudaErrorInvalidValue;
}

int fused_smem_bytes(int max_width) {
  const int tile = kDenseBlockRows * (max_width | 1) * 4;
  const int dense = kDProgBytes + dense_in_bytes() + align_up(tile, 16);
  return dense > kNgScratch ? dense : kNgScratch;
}

int fused_occupancy(int smem_bytes, int n_dense, int n_sparse, int* ctas_per_sm) {
  cudaError_t e;
  if (n_dense <= 32 && n_sparse <= 64) {
    e = cudaFuncSetAttribute(rap_fused_kernel<32, 64>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
    if (e == cudaSuccess)
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, rap_fused_kernel<32, 64>, kThreads, smem_bytes);
  } else {
    e = cudaFuncSetAttribute(rap_fused_kernel<128, 1024>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
    if (e == cudaSuccess)
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, rap_fused_kernel<128, 1024>, kThreads,
                                                        smem_bytes);
  }
  return (int)e;
}

}  // namespace rapk
