// rap_kernel.cu — the fused, persistent sm_100a preprocessing kernel.
//
// One launch processes a whole raw batch (§6.1: horizontal
// fusion of the per-feature kernels; here every op of every feature runs in a
// single persistent kernel, so the chains are fused vertically as well and no
// intermediate touches HBM).  CTAs pull (feature, row-range) descriptors from
// an atomic ticket counter.  Sparse descriptors come first, in feature-major
// order, and build the jagged offsets with a block scan plus a decoupled
// look-back across descriptors (the single-pass scan of DESIGN.md §7); dense
// descriptors transpose columnar input to the row-major MLP input through
// shared memory.  The grid is capped by the SM budget (§6.2).
//
// Operator semantics: DESIGN.md §3 readings R1-R20 (Table 1).
// Nothing here is tensor-core work: the path is integer ALU + a few SFU
// transcendentals, bound by HBM bandwidth.
#include <cuda_runtime.h>
#include <math.h>
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

// ----------------------------------------------------------------------------
// Scalar helpers.

__device__ __forceinline__ uint64_t reduce_M(uint64_t h, int64_t M) {  // R2
  return __umul64hi(h, (uint64_t)M);
}

__device__ __forceinline__ bool bit_valid(const uint32_t* bm, int64_t r) {  // R19
  if (bm == nullptr) return true;
  return (__ldg(bm + (r >> 5)) >> (r & 31)) & 1u;
}

__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_relaxed(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Upper bound = #{i : b[i] <= x} for sorted borders (R4; NaN -> 0).
__device__ __forceinline__ int64_t upper_bound_f(const float* b, int m, float x) {
  int lo = 0, n = m;
  while (n > 0) {
    int half = n >> 1;
    if (__ldg(b + lo + half) <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}

__device__ __forceinline__ int64_t upper_bound_i(const int64_t* b, int m, int64_t x) {
  int lo = 0, n = m;
  while (n > 0) {
    int half = n >> 1;
    if (__ldg(b + lo + half) <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}

// MapId (R8): keys sorted ascending at t[0..m), values at t[m..2m).
__device__ __forceinline__ int64_t map_lookup(const int64_t* t, int m, int64_t x, int64_t dflt) {
  int lo = 0, n = m;
  while (n > 0) {
    int half = n >> 1;
    if (__ldg(t + lo + half) < x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return (lo < m && __ldg(t + lo) == x) ? __ldg(t + m + lo) : dflt;
}

template <class P>
__device__ __forceinline__ int64_t apply_id_ops(const P& p, int64_t v, int o0, int o1) {
  for (int o = o0; o < o1; ++o) {
    const DevOp& op = p.c.ops[o];
    switch (op.kind) {
      case OK_CLAMP:  // R6
        v = v < op.a ? op.a : v;
        v = v > op.b ? op.b : v;
        break;
      case OK_SIGRID:  // R3: reduce(H(H(salt) ^ x), M)
        v = (int64_t)reduce_M(splitmix_H(op.hsalt ^ (uint64_t)v), op.M);
        break;
      case OK_BUCKET_I:
        v = upper_bound_i(p.c.itab + op.a, op.m, v);
        break;
      default:  // OK_MAPID
        v = map_lookup(p.c.itab + op.a, op.m, v, op.b);
        break;
    }
  }
  return v;
}

// Dense expression (R10-R12, R14): null slot -> NaN, then FillNull/Logit/BoxCox in f32.
template <class P>
__device__ float dense_expr(const P& p, int e, int64_t row) {
  const DenseExpr de = p.c.dexprs[e];
  float x = bit_valid(p.dvalid[de.col], row) ? __ldg(p.dense[de.col] + row) : __int_as_float(0x7fc00000);
  for (int o = de.op_begin; o < de.op_end; ++o) {
    const DevOp& op = p.c.ops[o];
    if (op.kind == OK_FILL_F) {
      if (isnan(x)) x = op.f0;
    } else if (op.kind == OK_LOGIT) {
      float z = x < op.f0 ? op.f0 : (x > op.f1 ? op.f1 : x);
      float q = __fdiv_rn(z, __fsub_rn(1.0f, z));
      x = logf(q);
    } else {  // OK_BOXCOX
      float lam = op.f0;
      if (lam == 0.0f) {
        x = logf(x);
      } else {
        float t = logf(x);
        float u = __fmul_rn(lam, t);
        x = __fdiv_rn(expm1f(u), lam);
      }
    }
  }
  return x;
}

// Per-row source description of a (non-NGram) chain.
struct RowSrc {
  int64_t start;  // first child index (mode 0)
  int64_t len;    // output length of the chain for this row
  int32_t mode;   // 0 = child values, 1 = filled null row, 2 = computed (dense bucket)
};

template <class P>
__device__ __forceinline__ RowSrc leaf_row(const P& p, const Chain& ch, int64_t row) {
  RowSrc r;
  if (ch.src_kind == SRC_SPARSE) {
    const int s = ch.src;
    if (bit_valid(p.svalid[s], row)) {
      const int64_t a = __ldg(p.off[s] + row), b = __ldg(p.off[s] + row + 1);
      r.start = a;
      r.len = min(max(b - a, (int64_t)0), ch.xcap);  // R5 FirstX as a cap
      r.mode = 0;
    } else {
      r.start = 0;
      r.mode = 1;
      r.len = ch.has_fill ? min((int64_t)1, ch.null_xcap) : 0;  // R10 / R14
    }
  } else {  // SRC_DENSE_BUCKET: always a length-1 list (R4)
    r.start = 0;
    r.mode = 2;
    r.len = min((int64_t)1, ch.xcap);
  }
  return r;
}

template <class P>
__device__ __forceinline__ int64_t leaf_elem(const P& p, const Chain& ch, const RowSrc& rs, int64_t row, int64_t j) {
  int64_t v;
  int o0;
  if (rs.mode == 0) {
    v = __ldg(p.val[ch.src] + rs.start + j);
    o0 = ch.op_begin;
  } else if (rs.mode == 1) {
    v = ch.fill;
    o0 = ch.null_op_begin;
  } else {
    v = upper_bound_f(p.c.ftab + ch.btab, ch.bm, dense_expr(p, ch.src, row));
    o0 = ch.op_begin;
  }
  return apply_id_ops(p, v, o0, ch.op_end);
}

// NGram (R7): count = max(0, sum_c len_c - n + 1).
template <class P>
__device__ int64_t ngram_row(const P& p, const NGramDesc& ng, int64_t row, RowSrc* rs) {
  int64_t tot = 0;
  for (int c = 0; c < ng.k; ++c) {
    rs[c] = leaf_row(p, p.c.chains[ng.chain[c]], row);
    tot += rs[c].len;
  }
  return max(tot - ng.n + 1, (int64_t)0);
}

template <class P>
__device__ int64_t ngram_elem(const P& p, const NGramDesc& ng, const RowSrc* rs, int64_t row, int64_t j) {
  uint64_t h = ng.hsalt;  // H(salt)
  int c = 0;
  int64_t pos = j;
  for (int i = 0; i < ng.n; ++i) {
    while (pos >= rs[c].len) {
      pos -= rs[c].len;
      ++c;
    }
    const int64_t e = leaf_elem(p, p.c.chains[ng.chain[c]], rs[c], row, pos);
    h = splitmix_H(h ^ (uint64_t)e);
    ++pos;
  }
  return (int64_t)reduce_M(h, ng.M);
}

template <class P>
__device__ __forceinline__ int64_t chain_row(const P& p, const Chain& ch, int64_t row, RowSrc* rs) {
  if (ch.src_kind != SRC_NGRAM) {
    rs[0] = leaf_row(p, ch, row);
    return rs[0].len;
  }
  return min(ngram_row(p, p.c.ngrams[ch.src], row, rs), ch.xcap);
}

template <class P>
__device__ __forceinline__ int64_t chain_elem(const P& p, const Chain& ch, const RowSrc* rs, int64_t row, int64_t j) {
  if (ch.src_kind != SRC_NGRAM) return leaf_elem(p, ch, rs[0], row, j);
  const int64_t v = ngram_elem(p, p.c.ngrams[ch.src], rs, row, j);
  return apply_id_ops(p, v, ch.op_begin, ch.op_end);
}

__device__ __forceinline__ long long warp_sum64(long long v) {
#pragma unroll
  for (int d = 16; d >= 1; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
  return v;
}

// Decoupled look-back (warp 0 of the CTA).  Publishes this descriptor's
// aggregate, walks predecessors 32 at a time until an inclusive prefix is
// found, publishes its own inclusive prefix, returns the exclusive prefix.
__device__ long long lookback(unsigned long long* status, long long slot, long long agg, unsigned long long epoch,
                              int lane) {
  const unsigned long long tag = epoch << kEpochShift;
  if (slot == 0) {
    if (lane == 0) st_relaxed(status, tag | (kFlagPrefix << kFlagShift) | (unsigned long long)agg);
    return 0;
  }
  if (lane == 0) st_relaxed(status + slot, tag | (kFlagAgg << kFlagShift) | (unsigned long long)agg);
  long long excl = 0;
  long long top = slot - 1;
  while (true) {
    const long long idx = top - lane;
    unsigned long long w = 0;
    int flag = (int)kFlagPrefix;  // before slot 0: an inclusive prefix of 0
    int spins = 0;
    while (true) {
      if (idx >= 0) {
        w = ld_relaxed(status + idx);
        flag = ((w >> kEpochShift) == epoch) ? (int)((w >> kFlagShift) & 3ull) : 0;
      }
      if (__all_sync(0xffffffffu, flag != 0)) break;
      if (++spins > 8) __nanosleep(64);
    }
    long long v = idx >= 0 ? (long long)(w & kValueMask) : 0;
    const unsigned pmask = __ballot_sync(0xffffffffu, flag == (int)kFlagPrefix);
    if (pmask) {
      const int first = __ffs(pmask) - 1;
      excl += warp_sum64(lane <= first ? v : 0);
      break;
    }
    excl += warp_sum64(v);
    top -= 32;
  }
  if (lane == 0) st_relaxed(status + slot, tag | (kFlagPrefix << kFlagShift) | (unsigned long long)(excl + agg));
  return excl;
}

struct SparseSmem {
  int32_t* len;
  int64_t* excl;
  int32_t* start;
};

__host__ __device__ constexpr int align_up(int x, int a) { return (x + a - 1) / a * a; }

// ----------------------------------------------------------------------------
// Sparse descriptor: (output feature f, rows [r0, r0+nr)).
template <class P>
__device__ void sparse_desc(const P& p, long long t, unsigned long long epoch, unsigned char* smem, long long* s_warp,
                            long long* s_bcast) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int kWarps = kThreads / 32;
  // feature = largest f with desc_start[f] <= t
  int lo = 0, n = p.c.n_sparse_out;
  while (n > 0) {
    int half = n >> 1;
    if (__ldg(p.c.desc_start + lo + half) <= t) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  const int f = lo - 1;
  const SparseOut so = p.c.souts[f];
  const Chain ch = p.c.chains[so.chain];
  const int64_t B = p.c.n_rows;
  const int64_t r0 = (t - __ldg(p.c.desc_start + f)) * (int64_t)so.rows_per_desc;
  const int nr = (int)min((int64_t)so.rows_per_desc, B - r0);
  const int R = so.rows_per_desc;
  int32_t* s_len = reinterpret_cast<int32_t*>(smem);
  int64_t* s_excl = reinterpret_cast<int64_t*>(smem + align_up(4 * R, 16));
  int32_t* s_start = reinterpret_cast<int32_t*>(smem + align_up(4 * R, 16) + 8 * R);

  // Phase A: closed-form output length of every row (a3).
  for (int i = tid; i < nr; i += kThreads) {
    const int64_t row = r0 + i;
    int64_t len;
    int32_t st = -1;
    if (ch.src_kind == SRC_SPARSE) {
      const RowSrc rs = leaf_row(p, ch, row);
      len = rs.len;
      st = rs.mode == 0 ? (int32_t)rs.start : -1;
    } else {
      RowSrc rs[kMaxNgramK];
      len = chain_row(p, ch, row, rs);
    }
    s_len[i] = (int32_t)len;
    s_start[i] = st;
  }
  __syncthreads();

  // Phase B: block exclusive scan (per-thread serial + warp shuffle + smem).
  const int per = (nr + kThreads - 1) / kThreads;
  long long local = 0;
  for (int k = 0; k < per; ++k) {
    const int i = tid * per + k;
    if (i < nr) local += s_len[i];
  }
  long long incl = local;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const long long y = __shfl_up_sync(0xffffffffu, incl, d);
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
    // Phase C: decoupled look-back across descriptors (slot = ticket).
    const long long excl = lookback(p.c.status, t, agg, epoch, lane);
    if (lane == 0) {
      s_bcast[0] = excl;
      s_bcast[1] = agg;
    }
  }
  __syncthreads();
  {
    long long run = s_warp[warp] + incl - local;
    for (int k = 0; k < per; ++k) {
      const int i = tid * per + k;
      if (i < nr) {
        s_excl[i] = run;
        run += s_len[i];
      }
    }
  }
  const long long base = s_bcast[0];
  const long long agg = s_bcast[1];
  __syncthreads();

  // Phase D: lengths / offsets (feature-major, R17).
  const int64_t fB = (int64_t)f * B;
  for (int i = tid; i < nr; i += kThreads) {
    p.c.lengths[fB + r0 + i] = s_len[i];
    p.c.offsets[fB + r0 + i] = base + s_excl[i];
  }
  if (tid == 0) {
    if (t == p.c.n_sparse_desc - 1) p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + agg;
    if (base + agg > p.c.values_cap) atomicExch(p.c.err, 1);
  }

  // Phase E: values, one warp per 32-row group, elements in output order.
  const int ngroups = (nr + 31) / 32;
  const long long cap = p.c.values_cap;
  for (int g = warp; g < ngroups; g += kWarps) {
    const int i = g * 32 + lane;
    const bool has = i < nr;
    const int len = has ? s_len[i] : 0;
    const long long ex = has ? s_excl[i] : 0;
    const long long gbase = __shfl_sync(0xffffffffu, ex, 0);
    const int lastlane = min(31, nr - 1 - g * 32);
    long long lex = ex - gbase;
    const long long T = __shfl_sync(0xffffffffu, lex + len, lastlane);
    if (!has) lex = LLONG_MAX;
    const long long out0 = base + gbase;
    if (__all_sync(0xffffffffu, !has || len == 1)) {
      // fast path: one id per row (single-valued Criteo features)
      if (has) {
        const int64_t row = r0 + i;
        int64_t v;
        if (ch.src_kind == SRC_SPARSE) {
          const int32_t st = s_start[i];
          v = st >= 0 ? apply_id_ops(p, __ldg(p.val[ch.src] + st), ch.op_begin, ch.op_end)
                      : apply_id_ops(p, ch.fill, ch.null_op_begin, ch.op_end);
        } else {
          RowSrc rs[kMaxNgramK];
          chain_row(p, ch, row, rs);
          v = chain_elem(p, ch, rs, row, 0);
        }
        const long long pos = out0 + lane;
        if (pos < cap) p.c.values[pos] = v;
      }
      continue;
    }
    for (long long eb = 0; eb < T; eb += 32) {
      const long long e = eb + lane;
      int r = 0;
#pragma unroll
      for (int step = 16; step >= 1; step >>= 1) {
        const long long c = __shfl_sync(0xffffffffu, lex, r + step);
        if (c <= e) r += step;
      }
      const long long lex_r = __shfl_sync(0xffffffffu, lex, r);
      if (e < T) {
        const int ii = g * 32 + r;
        const int64_t row = r0 + ii;
        const long long j = e - lex_r;
        int64_t v;
        if (ch.src_kind == SRC_SPARSE) {
          const int32_t st = s_start[ii];
          v = st >= 0 ? apply_id_ops(p, __ldg(p.val[ch.src] + st + j), ch.op_begin, ch.op_end)
                      : apply_id_ops(p, ch.fill, ch.null_op_begin, ch.op_end);
        } else {
          RowSrc rs[kMaxNgramK];
          chain_row(p, ch, row, rs);
          v = chain_elem(p, ch, rs, row, j);
        }
        const long long pos = out0 + e;
        if (pos < cap) p.c.values[pos] = v;
      }
    }
  }
}

// ----------------------------------------------------------------------------
// Dense descriptor: (row block, column group) -> row-major tile via smem (a2).
template <class P>
__device__ void dense_desc(const P& p, long long t, unsigned char* smem) {
  const int tid = threadIdx.x;
  const int gi = (int)(t % p.c.n_groups);
  const long long rb = t / p.c.n_groups;
  const Group g = p.c.groups[gi];
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rb * (int64_t)p.c.rows_dense;
  const int nr = (int)min((int64_t)p.c.rows_dense, B - r0);
  const int LD = p.c.tile_ld;
  const int W = g.width;
  float* tile = reinterpret_cast<float*>(smem);
  for (int i = tid; i < nr * LD; i += kThreads) tile[i] = 0.0f;
  __syncthreads();
  for (int u = g.unit_begin; u < g.unit_end; ++u) {
    const Unit un = p.c.units[u];
    const int c = un.col - g.col0;
    if (un.kind == U_DENSE) {
      for (int r = tid; r < nr; r += kThreads) tile[r * LD + c] = dense_expr(p, un.idx, r0 + r);
    } else {  // OneHot columns [col, col+width) <-> ids [k0, k0+width) (R9)
      const Chain ch = p.c.chains[un.idx];
      for (int r = tid; r < nr; r += kThreads) {
        const int64_t row = r0 + r;
        RowSrc rs[kMaxNgramK];
        const int64_t L = chain_row(p, ch, row, rs);
        for (int64_t j = 0; j < L; ++j) {
          const int64_t d = chain_elem(p, ch, rs, row, j) - un.k0;
          if (d >= 0 && d < un.width) tile[r * LD + c + (int)d] = 1.0f;
        }
      }
    }
  }
  __syncthreads();
  float* out = p.c.dense_out + r0 * p.c.ld + g.col0;
  const int64_t ld = p.c.ld;
  for (int i = tid; i < nr * W; i += kThreads) {
    const int r = i / W;
    const int cc = i - r * W;
    out[r * ld + cc] = tile[r * LD + cc];
  }
}

template <int MD, int MS>
__global__ void __launch_bounds__(kThreads) rap_fused_kernel(const __grid_constant__ KParams<MD, MS> p) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ long long s_ticket;
  __shared__ unsigned long long s_epoch;
  __shared__ int s_last;
  __shared__ long long s_warp[kThreads / 32];
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
      sparse_desc(p, t, epoch, smem, s_warp, s_bcast);
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
