// rap_kernel.cu — the fused, persistent sm_100a preprocessing kernel.
//
// One launch processes a whole raw batch (§6.1: horizontal
// fusion of the per-feature kernels; here every op of every feature runs in a
// single persistent kernel, so the chains are fused vertically as well and no
// intermediate touches HBM).  CTAs pull (feature, row-range) descriptors from
// an atomic ticket counter and copy the descriptor's flattened program
// (rap_internal.h) into shared memory in one burst.  Sparse descriptors come
// first, in feature-major order, and build the jagged offsets with a block
// scan plus a decoupled look-back across descriptors.  The
// look-back is deferred: a descriptor publishes its aggregate right after the
// length pass, computes its ids into shared memory, and only then asks for
// its prefix.  Dense descriptors transpose columnar input to the row-major
// MLP input through shared memory.  The grid is capped by the SM budget
// (§6.2).
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

__host__ __device__ constexpr int align_up(int x, int a) { return (x + a - 1) / a * a; }

// Shared-memory carve-up.  Sparse and dense descriptors reuse the same bytes.
constexpr int kSProgBytes = align_up((int)sizeof(SProg), 16);
constexpr int kSparseSmem = kSProgBytes + 8 * kStageTab + 8 * kVBuf + 3 * 4 * kRowsSparseMax + 2 * 4 * kNgSlots;
constexpr int kDProgBytes = align_up((int)sizeof(DProg), 16);

// ----------------------------------------------------------------------------
// Scalar helpers.

__device__ __forceinline__ uint64_t reduce_M(uint64_t h, int64_t M) {  // R2
  return __umul64hi(h, (uint64_t)M);
}

__device__ __forceinline__ uint32_t bitmap_word(const uint32_t* bm, int64_t r) {
  return bm == nullptr ? 0xffffffffu : __ldg(bm + (r >> 5));
}

__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_relaxed(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Upper bound = #{i : b[i] <= x} for sorted borders (R4; NaN -> 0).  Works on
// shared or global memory (generic pointer).
template <class T>
__device__ __forceinline__ int64_t upper_bound(const T* b, int m, T x) {
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
// linear probing.  A real INT64_MIN key is carried in the op itself.
__device__ __forceinline__ int64_t map_lookup(const DevOp& op, const int64_t* itab, int64_t x) {
  if (x == INT64_MIN) return op.M ? (int64_t)op.hsalt : op.b;
  const longlong2* t = reinterpret_cast<const longlong2*>(itab + op.a);
  const uint32_t mask = (1u << op.m) - 1u;
  uint32_t i = (uint32_t)(((uint64_t)x * 0x9E3779B97F4A7C15ull) >> (64 - op.m));
  while (true) {
    const longlong2 kv = __ldg(t + i);
    if (kv.x == x) return kv.y;
    if (kv.x == INT64_MIN) return op.b;
    i = (i + 1) & mask;
  }
}

__device__ __forceinline__ int64_t apply_id_ops(const DevOp* ops, const int64_t* itab, const int64_t* stab,
                                                int64_t v, int o0, int o1) {
  for (int o = o0; o < o1; ++o) {
    const DevOp& op = ops[o];
    switch (op.kind) {
      case OK_CLAMP:  // R6
        v = v < op.a ? op.a : v;
        v = v > op.b ? op.b : v;
        break;
      case OK_SIGRID:  // R3: reduce(H(H(salt) ^ x), M)
        v = (int64_t)reduce_M(splitmix_H(op.hsalt ^ (uint64_t)v), op.M);
        break;
      case OK_BUCKET_S:
        v = upper_bound(stab + op.a, op.m, v);
        break;
      case OK_BUCKET_I:
        v = upper_bound(itab + op.a, op.m, v);
        break;
      default:  // OK_MAPID
        v = map_lookup(op, itab, v);
        break;
    }
  }
  return v;
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

// Raw dense value with the R14 null rule (null slot -> NaN).
template <class P>
__device__ __forceinline__ float dense_raw(const P& p, int col, int64_t row) {
  const uint32_t w = bitmap_word(p.dvalid[col], row);
  const float x = __ldg(p.dense[col] + row);
  return ((w >> (row & 31)) & 1u) ? x : __int_as_float(0x7fc00000);
}

// ----------------------------------------------------------------------------
// Id-list chains.

// Source list of a chain for one row: returns the output length and the first
// child index (start >= 0), -1 for a filled null row, -2 for a dense bucket.
template <class P>
__device__ __forceinline__ int32_t leaf_len(const P& p, const Chain& ch, int64_t row, int32_t* start) {
  if (ch.src_kind == SRC_SPARSE) {
    const int s = ch.src;
    const uint32_t w = bitmap_word(p.svalid[s], row);
    const int32_t a = __ldg(p.off[s] + row), b = __ldg(p.off[s] + row + 1);
    if ((w >> (row & 31)) & 1u) {
      *start = a;
      return (int32_t)min((int64_t)max(b - a, 0), ch.xcap);  // R5 FirstX as a cap
    }
    *start = -1;
    return ch.has_fill ? (int32_t)min((int64_t)1, ch.null_xcap) : 0;  // R10 / R14
  }
  *start = -2;  // SRC_DENSE_BUCKET: always a length-1 list (R4)
  return (int32_t)min((int64_t)1, ch.xcap);
}

template <class P>
__device__ __forceinline__ int64_t leaf_value(const P& p, const DevOp* ops, const int64_t* stab, const Chain& ch,
                                              int32_t start, int64_t row, int32_t j) {
  if (start >= 0)
    return apply_id_ops(ops, p.c.itab, stab, __ldg(p.val[ch.src] + start + j), ch.op_begin, ch.op_end);
  if (start == -1) return apply_id_ops(ops, p.c.itab, stab, ch.fill, ch.null_op_begin, ch.op_end);
  const float x = apply_dense_ops(ops, dense_raw(p, ch.src, row), ch.dop_begin, ch.dop_end);
  return apply_id_ops(ops, p.c.itab, stab, upper_bound(p.c.ftab + ch.btab, ch.bm, x), ch.op_begin, ch.op_end);
}

__device__ __forceinline__ const DevOp* prog_ops(const SProg& pg, const DevOp* gops) {
  return pg.global_ops ? gops : pg.ops;
}

// Whole-chain length / element for any source kind (NGram sources
// recomputed from global memory), used by the OneHot generic unit.
template <class P>
__device__ int32_t chain_len_g(const P& p, const SProg& pg, int64_t row, int32_t* st, int32_t* sl) {
  if (pg.ch.src_kind != SRC_NGRAM) return leaf_len(p, pg.ch, row, st);
  int tot = 0;
  for (int c = 0; c < pg.ng.k; ++c) {
    sl[c] = leaf_len(p, pg.src[c], row, st + c);
    tot += sl[c];
  }
  return (int32_t)min((int64_t)max(tot - pg.ng.n + 1, 0), pg.ch.xcap);
}

template <class P>
__device__ int64_t ngram_window(const P& p, const SProg& pg, const DevOp* ops, const int64_t* stab, const int32_t* st,
                                const int32_t* sl, int stride, int64_t row, int32_t j) {
  // R7: h = H(salt); h = H(h ^ c[j+q]) for q < n; reduce(h, M)
  const NGramDesc& ng = pg.ng;
  uint64_t h = ng.hsalt;
  int c = 0;
  int32_t pos = j;
  int32_t lc = sl[0];
  for (int q = 0; q < ng.n; ++q) {
    while (pos >= lc) {
      pos -= lc;
      ++c;
      lc = sl[c * stride];
    }
    const int64_t e = leaf_value(p, ops, stab, pg.src[c], st[c * stride], row, pos);
    h = splitmix_H(h ^ (uint64_t)e);
    ++pos;
  }
  return apply_id_ops(ops, p.c.itab, stab, (int64_t)reduce_M(h, ng.M), pg.ch.op_begin, pg.ch.op_end);
}

template <class P>
__device__ int64_t chain_elem_g(const P& p, const SProg& pg, const int64_t* stab, const int32_t* st,
                                const int32_t* sl, int64_t row, int32_t j) {
  const DevOp* ops = prog_ops(pg, p.c.ops);
  if (pg.ch.src_kind != SRC_NGRAM) return leaf_value(p, ops, stab, pg.ch, st[0], row, j);
  return ngram_window(p, pg, ops, stab, st, sl, 1, row, j);
}

// ----------------------------------------------------------------------------
__device__ __forceinline__ long long warp_sum64(long long v) {
#pragma unroll
  for (int d = 16; d >= 1; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
  return v;
}

// Decoupled look-back (warp 0).  Each lane inspects 4 predecessor words, so
// one round trip covers 128 descriptors.  Walking from the nearest
// predecessor down, aggregates are summed until the first inclusive prefix;
// only an unpublished word on that path makes the warp wait (the part before
// it is banked).  Returns the exclusive prefix, publishes the inclusive one.
__device__ long long lookback(unsigned long long* status, long long slot, long long agg, unsigned long long epoch,
                              int lane) {
  const unsigned long long tag = epoch << kEpochShift;
  long long excl = 0;
  long long top = slot - 1;
  int spins = 0;
  while (top >= 0) {
    unsigned long long w[4];
    int flag[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const long long idx = top - 4 * lane - q;
      w[q] = idx >= 0 ? ld_relaxed(status + idx) : 0ull;
      flag[q] = idx >= 0 ? (((w[q] >> kEpochShift) == epoch) ? (int)((w[q] >> kFlagShift) & 3ull) : 0)
                         : (int)kFlagPrefix;
    }
    int qstop = 4;  // first slot (descending) that is unpublished or a prefix
#pragma unroll
    for (int q = 3; q >= 0; --q)
      if (flag[q] != (int)kFlagAgg) qstop = q;
    const unsigned smask = __ballot_sync(0xffffffffu, qstop < 4);
    const int fl = smask ? __ffs(smask) - 1 : 32;
    const int fq = __shfl_sync(0xffffffffu, qstop, fl & 31);
    int mykind = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q)
      if (q == qstop) mykind = flag[q];
    const int fkind = __shfl_sync(0xffffffffu, mykind, fl & 31);
    long long v = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const bool take = lane < fl || (lane == fl && (q < fq || (q == fq && fkind == (int)kFlagPrefix)));
      if (take) v += (long long)(w[q] & kValueMask);
    }
    excl += warp_sum64(v);
    if (smask == 0) {
      top -= 128;
      continue;
    }
    if (fkind == (int)kFlagPrefix) break;
    top -= 4 * fl + fq;  // wait on the first unpublished predecessor
    if (++spins > 2) __nanosleep(32);
  }
  if (lane == 0) st_relaxed(status + slot, tag | (kFlagPrefix << kFlagShift) | (unsigned long long)(excl + agg));
  return excl;
}

// Warp-cooperative 16-byte copy global -> shared.
__device__ __forceinline__ void warp_copy16(void* dst, const void* src, int bytes, int lane) {
  const int4* s = reinterpret_cast<const int4*>(src);
  int4* d = reinterpret_cast<int4*>(dst);
  const int n = bytes >> 4;
  for (int k = lane; k < n; k += 32) d[k] = __ldg(s + k);
}

struct SparseSmem {
  SProg* prog;
  int64_t* tab;    // [kStageTab] staged Bucketize borders
  int64_t* vals;   // [kVBuf] staged output ids
  int32_t* len;    // [R] output length per row
  int32_t* excl;   // [R] exclusive prefix within the descriptor
  int32_t* start;  // [R] first child index (-1 filled null row, -2 computed)
  int32_t* ngs;    // [kNgSlots] NGram: per (source, row) start
  int32_t* ngl;    // [kNgSlots] NGram: per (source, row) length
};

__device__ __forceinline__ SparseSmem carve_sparse(unsigned char* smem) {
  SparseSmem s;
  int o = 0;
  s.prog = reinterpret_cast<SProg*>(smem + o);
  o += kSProgBytes;
  s.tab = reinterpret_cast<int64_t*>(smem + o);
  o += 8 * kStageTab;
  s.vals = reinterpret_cast<int64_t*>(smem + o);
  o += 8 * kVBuf;
  s.len = reinterpret_cast<int32_t*>(smem + o);
  o += 4 * kRowsSparseMax;
  s.excl = reinterpret_cast<int32_t*>(smem + o);
  o += 4 * kRowsSparseMax;
  s.start = reinterpret_cast<int32_t*>(smem + o);
  o += 4 * kRowsSparseMax;
  s.ngs = reinterpret_cast<int32_t*>(smem + o);
  o += 4 * kNgSlots;
  s.ngl = reinterpret_cast<int32_t*>(smem + o);
  return s;
}

// Warp 0: feature of ticket t by a 32-ary search over desc_start (one round
// trip for <= 32 features, two for <= 1024), then the program copy.
template <class P>
__device__ int locate_and_stage(const P& p, long long t, const SparseSmem& sm) {
  const int lane = threadIdx.x & 31;
  int lo = 0, hi = p.c.n_sparse_out;
  while (hi - lo > 1) {
    const int step = (hi - lo + 31) >> 5;
    const int idx = lo + lane * step;
    const bool ok = idx < hi && __ldg(p.c.desc_start + idx) <= t;
    const unsigned m = __ballot_sync(0xffffffffu, ok);
    const int k = 31 - __clz(m);
    lo += k * step;
    hi = min(hi, lo + step);
  }
  const int f = lo;
  const SProg* g = p.c.sprogs + f;
  warp_copy16(sm.prog, g, kSProgBytes, lane);
  __syncwarp();
  const int tl = sm.prog->tab_len;
  if (tl > 0) warp_copy16(sm.tab, p.c.itab + sm.prog->tab_off, align_up(8 * tl, 16), lane);
  return f;
}

// Value of output element j of local row i.
template <class P>
__device__ __forceinline__ int64_t sparse_value(const P& p, const SProg& pg, const DevOp* ops, const SparseSmem& sm,
                                                int R, int64_t r0, int i, int32_t j) {
  if (pg.ch.src_kind != SRC_NGRAM) return leaf_value(p, ops, sm.tab, pg.ch, sm.start[i], r0 + i, j);
  return ngram_window(p, pg, ops, sm.tab, sm.ngs + i, sm.ngl + i, R, r0 + i, j);
}

// Elements of a descriptor, one warp per 32-row group, emitted into shared
// memory or straight to the output (dst already offset by the base).
template <class P>
__device__ void emit_values(const P& p, const SProg& pg, const DevOp* ops, const SparseSmem& sm, int R, int64_t r0,
                            int nr, int64_t* dst, long long dst_limit) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int ngroups = (nr + 31) / 32;
  for (int g = warp; g < ngroups; g += kWarps) {
    const int i = g * 32 + lane;
    const bool has = i < nr;
    const int len = has ? sm.len[i] : 0;
    const int ex = has ? sm.excl[i] : 0;
    const int gbase = __shfl_sync(0xffffffffu, ex, 0);
    const int lastlane = min(31, nr - 1 - g * 32);
    int lex = ex - gbase;
    const int T = __shfl_sync(0xffffffffu, lex + len, lastlane);
    if (!has) lex = INT_MAX;
    int64_t* out = dst + gbase;
    const long long lim = dst_limit - gbase;
    if (__all_sync(0xffffffffu, !has || len == 1)) {
      if (has && lane < lim) out[lane] = sparse_value(p, pg, ops, sm, R, r0, i, 0);
      continue;
    }
    for (int eb = 0; eb < T; eb += 32) {
      const int e = eb + lane;
      int r = 0;
#pragma unroll
      for (int step = 16; step >= 1; step >>= 1) {
        const int c = __shfl_sync(0xffffffffu, lex, r + step);
        if (c <= e) r += step;
      }
      const int lex_r = __shfl_sync(0xffffffffu, lex, r);
      if (e < T && e < lim) out[e] = sparse_value(p, pg, ops, sm, R, r0, g * 32 + r, e - lex_r);
    }
  }
}

// ----------------------------------------------------------------------------
// Sparse descriptor: (output feature f, rows [r0, r0+nr)).
template <class P>
__device__ void sparse_desc(const P& p, long long t, unsigned long long epoch, unsigned char* smem, long long* s_warp,
                            long long* s_bcast, int* s_f) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const SparseSmem sm = carve_sparse(smem);
  if (warp == 0) {
    const int f = locate_and_stage(p, t, sm);
    if (lane == 0) *s_f = f;
  }
  __syncthreads();
  const int f = *s_f;
  const SProg& pg = *sm.prog;
  const DevOp* ops = prog_ops(pg, p.c.ops);
  const int R = __ldg(p.c.rows_per_desc + f);
  const int64_t B = p.c.n_rows;
  const int64_t r0 = (t - __ldg(p.c.desc_start + f)) * (int64_t)R;
  const int nr = (int)min((int64_t)R, B - r0);

  // Phase A: closed-form output length of every row (a3).  Each thread owns
  // `per` consecutive rows; all loads of a row are issued together.
  const int per = (R + kThreads - 1) / kThreads;
  const int i0 = tid * per;
  int local = 0;
  if (pg.ch.src_kind != SRC_NGRAM) {
#pragma unroll 4
    for (int k = 0; k < per; ++k) {
      const int i = i0 + k;
      if (i < nr) {
        int32_t st;
        const int32_t len = leaf_len(p, pg.ch, r0 + i, &st);
        sm.len[i] = len;
        sm.start[i] = st;
        local += len;
      }
    }
  } else {
    for (int k = 0; k < per; ++k) {
      const int i = i0 + k;
      if (i < nr) {
        int tot = 0;
#pragma unroll 4
        for (int c = 0; c < pg.ng.k; ++c) {
          int32_t st;
          const int32_t lc = leaf_len(p, pg.src[c], r0 + i, &st);
          sm.ngs[c * R + i] = st;
          sm.ngl[c * R + i] = lc;
          tot += lc;
        }
        const int32_t len = (int32_t)min((int64_t)max(tot - pg.ng.n + 1, 0), pg.ch.xcap);
        sm.len[i] = len;
        local += len;
      }
    }
  }
  // Phase B: block exclusive scan (warp shuffle + smem); aggregate published early.
  int incl = local;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, incl, d);
    if (lane >= d) incl += y;
  }
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const long long w = lane < kWarps ? s_warp[lane] : 0;
    long long wi = w;
#pragma unroll
    for (int d = 1; d < kWarps; d <<= 1) {
      const long long y = __shfl_up_sync(0xffffffffu, wi, d);
      if (lane >= d) wi += y;
    }
    const long long agg = __shfl_sync(0xffffffffu, wi, kWarps - 1);
    if (lane < kWarps) s_warp[lane] = wi - w;
    if (lane == 0) {
      s_bcast[1] = agg;
      const unsigned long long tag = epoch << kEpochShift;
      st_relaxed(p.c.status + t, tag | ((t == 0 ? kFlagPrefix : kFlagAgg) << kFlagShift) | (unsigned long long)agg);
    }
  }
  __syncthreads();
  {
    int run = (int)s_warp[warp] + incl - local;
    for (int k = 0; k < per; ++k) {
      const int i = i0 + k;
      if (i < nr) {
        sm.excl[i] = run;
        run += sm.len[i];
      }
    }
  }
  const long long agg = s_bcast[1];
  __syncthreads();

  const bool staged = agg <= kVBuf;
  if (staged) {
    // Phase E (ids into shared memory) while predecessors resolve their prefixes.
    emit_values(p, pg, ops, sm, R, r0, nr, sm.vals, LLONG_MAX);
  }
  // Phase C: decoupled look-back (slot = ticket).
  if (warp == 0) {
    const long long excl = t == 0 ? 0 : lookback(p.c.status, t, agg, epoch, lane);
    if (lane == 0) s_bcast[0] = excl;
  }
  __syncthreads();
  const long long base = s_bcast[0];

  // Phase D: lengths / offsets (feature-major, R17), then the ids.
  const int64_t fB = (int64_t)f * B + r0;
  for (int i = tid; i < nr; i += kThreads) {
    p.c.lengths[fB + i] = sm.len[i];
    p.c.offsets[fB + i] = base + sm.excl[i];
  }
  if (tid == 0) {
    if (t == p.c.n_sparse_desc - 1) p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + agg;
    if (base + agg > p.c.values_cap) atomicExch(p.c.err, 1);
  }
  const long long cap = p.c.values_cap;
  if (staged) {
    int64_t* out = p.c.values + base;
    const int lim = (int)min(agg, cap - base);
    for (int k = tid; k < lim; k += kThreads) out[k] = sm.vals[k];
  } else {
    emit_values(p, pg, ops, sm, R, r0, nr, p.c.values + base, cap - base);
  }
}

// ----------------------------------------------------------------------------
// Dense descriptor: (row block, column group) -> row-major tile via smem (a2).
template <class P>
__device__ void dense_desc(const P& p, long long t, unsigned char* smem) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int gi = (int)(t % p.c.n_groups);
  const long long rb = t / p.c.n_groups;
  DProg* dp = reinterpret_cast<DProg*>(smem);
  float* tile = reinterpret_cast<float*>(smem + kDProgBytes);
  if (warp == 0) {
    // header + used units, used ops, used borders
    const DProg* g = p.c.dprogs + gi;
    const int nu = __ldg(&g->n_units), no = __ldg(&g->n_ops), nf = __ldg(&g->n_ftab);
    warp_copy16(dp, g, align_up((int)offsetof(DProg, units) + nu * (int)sizeof(DUnit), 16), lane);
    warp_copy16(dp->ops, g->ops, align_up(no * (int)sizeof(DevOp), 16), lane);
    warp_copy16(dp->ftab, g->ftab, align_up(nf * 4, 16), lane);
  }
  __syncthreads();
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rb * (int64_t)p.c.rows_dense;
  const int nr = (int)min((int64_t)p.c.rows_dense, B - r0);
  const int W = dp->width;
  const int LD = W | 1;  // odd row pitch: conflict-free column writes
  if (dp->any_onehot) {
    for (int i = tid; i < nr * LD; i += kThreads) tile[i] = 0.0f;
    __syncthreads();
  }
  const int nu = dp->n_units;
  for (int r = tid; r < nr; r += kThreads) {
    const int64_t row = r0 + r;
    for (int u = 0; u < nu; ++u) {
      const DUnit& un = dp->units[u];
      const DevOp* uops = un.gops ? p.c.ops : dp->ops;
      if (un.kind == U_DENSE) {
        tile[r * LD + un.col] = apply_dense_ops(uops, dense_raw(p, un.src_col, row), un.op_begin, un.op_end);
      } else if (un.kind == U_ONEHOT_DB) {
        if (un.xcap > 0) {
          const float* uft = un.gops ? p.c.ftab : dp->ftab;
          const float x = apply_dense_ops(uops, dense_raw(p, un.src_col, row), un.op_begin, un.op_end);
          const int64_t id = apply_id_ops(uops, p.c.itab, nullptr, upper_bound(uft + un.btab, un.bm, x),
                                          un.iop_begin, un.iop_end);
          const int64_t d = id - un.k0;
          if (d >= 0 && d < un.width) tile[r * LD + un.col + (int)d] = 1.0f;
        }
      } else {  // U_ONEHOT_G: generic list (R9), program read from global memory
        const SProg& pg = p.c.oprogs[un.prog];
        const int64_t* stab = p.c.itab + pg.tab_off;
        int32_t st[kMaxNgramK], sl[kMaxNgramK];
        const int32_t L = chain_len_g(p, pg, row, st, sl);
        for (int32_t j = 0; j < L; ++j) {
          const int64_t d = chain_elem_g(p, pg, stab, st, sl, row, j) - un.k0;
          if (d >= 0 && d < un.width) tile[r * LD + un.col + (int)d] = 1.0f;
        }
      }
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
}

template <int MD, int MS>
__global__ void __launch_bounds__(kThreads, 4) rap_fused_kernel(const __grid_constant__ KParams<MD, MS> p) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ long long s_ticket;
  __shared__ unsigned long long s_epoch;
  __shared__ int s_last;
  __shared__ int s_f;
  __shared__ long long s_warp[kWarps];
  __shared__ long long s_bcast[2];
  const int tid = threadIdx.x;
  unsigned long long* sched = p.c.sched;
  if (tid == 0) {
    s_epoch = ld_relaxed(sched + 2);
    s_ticket = (long long)atomicAdd(sched, 1ull);
  }
  __syncthreads();
  const unsigned long long epoch = s_epoch;
  long long t = s_ticket;
  while (t < p.c.n_total_desc) {
    unsigned long long nxt = 0;
    if (tid == 0) nxt = atomicAdd(sched, 1ull);  // prefetch the next ticket
    if (t < p.c.n_sparse_desc) {
      sparse_desc(p, t, epoch, smem, s_warp, s_bcast, &s_f);
    } else {
      dense_desc(p, t - p.c.n_sparse_desc, smem);
    }
    __syncthreads();
    if (tid == 0) s_ticket = (long long)nxt;
    __syncthreads();
    t = s_ticket;
  }
  // The last CTA out resets the ticket / done counters and advances the epoch
  // (clearing the look-back words when the 20-bit epoch wraps).
  if (tid == 0) {
    __threadfence();
    const unsigned long long prev = atomicAdd(sched + 1, 1ull);
    s_last = (prev == (unsigned long long)gridDim.x - 1) ? 1 : 0;
    if (s_last) __threadfence();
  }
  __syncthreads();
  if (s_last) {
    const bool wrap = epoch >= kEpochMax;
    if (wrap) {
      for (long long i = tid; i < p.c.status_cap; i += kThreads) p.c.status[i] = 0ull;
      __threadfence();
    }
    __syncthreads();
    if (tid == 0) {
      sched[0] = 0ull;
      sched[1] = 0ull;
      sched[2] = wrap ? 1ull : epoch + 1ull;
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
  rap_fused_kernel<MD, MS><<<grid, kThreads, smem, st>>>(p);
  return (int)cudaGetLastError();
}

int launch_fused(const Common& c, const LaunchRaw& raw, int grid, int smem_bytes, void* stream) {
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (raw.n_dense <= 32 && raw.n_sparse <= 64) return launch_t<32, 64>(c, raw, grid, smem_bytes, st);
  if (raw.n_dense <= 128 && raw.n_sparse <= 1024) return launch_t<128, 1024>(c, raw, grid, smem_bytes, st);
  return (int)cudaErrorInvalidValue;
}

int fused_smem_bytes(int tile_bytes) {
  const int dense = kDProgBytes + align_up(tile_bytes, 16);
  return dense > kSparseSmem ? dense : kSparseSmem;
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
