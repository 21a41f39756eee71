// rap_rows.cu — the row-block fused preprocessing kernel (sm_100a).
//
// One cooperative launch turns a raw columnar batch into the "input
// tensors" by evaluating every output's operator chain
// (Table 1; DAG per feature, L718-720): horizontal fusion across
// features and vertical fusion along each chain in one kernel (§6.1
// L1161-1174), intermediates never leave the SM.  It is the kernel the planner
// picks for Criteo-shaped batches (short id lists); rap_kernel.cu's tiled
// kernel handles long multi-hot lists element-parallel.
//
// Work: the rows are split into n_rb contiguous row blocks and the sparse
// outputs into n_fg feature groups (contiguous ranges of a processing order);
// CTA (g, r) evaluates group g over row block r, one row per thread, in
// 256-row chunks:
//   (1) lengths: the Arrow offsets and validity words of every raw column the
//       group reads are staged in shared memory with cp.async; each output's
//       row length is a closed form of them (R5, R7, R10, R14), cached in
//       shared memory; the per-output totals over the block are stored to
//       agg[f * n_rb + r] and a release counter announces the CTA;
//   (2) dense: the launch's dense blocks (FillNull / Logit / BoxCox /
//       Bucketize -> OneHot, row-major through a shared-memory tile), round
//       robin over the CTAs; they hide the wait of (3);
//   (3) base: once every CTA is announced, each warp reduces the totals of a
//       few outputs (all row blocks in parallel); every output's first offset
//       for this block is the feature-major exclusive prefix (R17);
//   (4) ids: per output, a warp scan gives each row its position; each
//       thread runs its row's list through the output's chain (Canon stages,
//       parameters in shared memory) and stores ids, lengths and offsets; the
//       next output's first id is loaded while the current one hashes.  A
//       canonical output memoises element 0 after a prefix of its stages, so
//       NGram windows over that prefix (C2's trigrams over post-SigridHash
//       sources) reuse it instead of re-hashing.
// The last CTA out resets the counters, so launch parameters are the same
// from call to call (CUDA-graph replayable).  The grid is capped by the SM
// budget (§6.2).
#include <cuda_runtime.h>
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#include <string.h>

#include "rap_internal.h"
#include "rap_device.cuh"

namespace rapk {

template <int MD, int MS>
struct RbParams {
  Common c;
  RbGeom g;
  const float* dense[MD];
  const uint32_t* dvalid[MD];
  const int32_t* off[MS];
  const int64_t* val[MS];
  const uint32_t* svalid[MS];
};

constexpr int kRbPitch = kRbChunk + 4;  // staged offsets of one column (257 used), 16-byte rows
constexpr uint32_t kLenBig = 0xffffu;   // cached length >= this: recompute

// Shared-memory record of one output of the CTA's group (built at CTA start
// from RbFeat and the output's SProg).
struct RbF {
  int32_t kind, emit, n, k;
  int32_t out_cap, memo_slot, memo_mask, f;
  int32_t cap[kMaxNgramK];
  int32_t ncap[kMaxNgramK];
  int16_t slot[kMaxNgramK];  // staged slot of source i (-1: dense-bucket source)
  int16_t prov[kMaxNgramK];  // NGram source i: processing index of its memo provider (-1: none)
  int16_t pslot[kMaxNgramK]; // ... and the provider's memo slot
  int64_t fill;              // emit 0: a filled null row's id (R10)
  int32_t src0;              // emit 0: raw column of the list
  int32_t memo_after;        // emit 0: memoise after this stage bit (16: before any stage, -1: no memo)
  Canon cn;                  // emit 0: the chain's stages (NGram: post-hash stages)
};

// Dynamic shared memory layout (rows_smem_bytes computes the same sizes).
struct RbSmem {
  unsigned char* dense;  // dense_block's region; phase (3) reductions and phase (4) memo reuse it
  RbF* feat;             // [max_fl]
  int32_t* off;          // [max_cols][kRbPitch] staged offsets of the chunk
  uint32_t* bm;          // [max_cols][8] staged validity words
  uint16_t* len;         // [max_fl][kRbChunk] lengths of the chunk (kLenBig: recompute)
  long long* ws;         // [max_fl][8] warp sums of the chunk
  long long* wb;         // [max_fl][8] warp bases of the chunk
  long long* base;       // [max_fl] running base (first offset of the next chunk)
  long long* memo;       // [n_memo][kRbChunk] memoised element 0 (phase 4)
};

__host__ __device__ inline int rb_align(int x) { return (x + 15) & ~15; }

__host__ __device__ inline int rb_region0(int dense_bytes, int n_memo, int max_f) {
  const int m = n_memo * kRbChunk * 8, r = 2 * (max_f + 1) * 8;
  return rb_align(dense_bytes > m ? (dense_bytes > r ? dense_bytes : r) : (m > r ? m : r));
}

__device__ __forceinline__ RbSmem rb_carve(unsigned char* smem, const RbGeom& g, int n_sparse_out) {
  RbSmem s;
  int o = rb_region0(g.dense_bytes, g.n_memo, n_sparse_out);
  s.dense = smem;
  s.memo = reinterpret_cast<long long*>(smem);
  s.ws = reinterpret_cast<long long*>(smem + o);
  o += rb_align(g.max_fl * 8 * 8);
  s.wb = reinterpret_cast<long long*>(smem + o);
  o += rb_align(g.max_fl * 8 * 8);
  s.base = reinterpret_cast<long long*>(smem + o);
  o += rb_align(g.max_fl * 8);
  s.feat = reinterpret_cast<RbF*>(smem + o);
  o += rb_align(g.max_fl * (int)sizeof(RbF));
  s.off = reinterpret_cast<int32_t*>(smem + o);
  o += rb_align(g.max_cols * kRbPitch * 4);
  s.bm = reinterpret_cast<uint32_t*>(smem + o);
  o += rb_align(g.max_cols * 8 * 4);
  s.len = reinterpret_cast<uint16_t*>(smem + o);
  return s;
}

__device__ __forceinline__ long long ld_cg64(const unsigned long long* p) {
  long long v;
  asm volatile("ld.global.cg.s64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

// ---- warp-level sums and scans (32-bit when every offset fits, R17) ----
template <bool kSmall>
__device__ __forceinline__ long long rb_warp_sum(long long v) {
  if (kSmall) return (long long)__reduce_add_sync(0xffffffffu, (unsigned)v);
  return warp_sum64(v);
}

template <bool kSmall>
__device__ __forceinline__ long long rb_warp_excl(int32_t v, int lane) {
  if (kSmall) {
    int x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, x, d);
      if (lane >= d) x += y;
    }
    return (long long)(x - v);
  }
  long long x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const long long y = __shfl_up_sync(0xffffffffu, x, d);
    if (lane >= d) x += y;
  }
  return x - v;
}

// ---- staged raw rows ----
struct RbRow {
  int32_t a, b;
  bool valid;
};

__device__ __forceinline__ RbRow rb_row(const RbSmem& s, int slot, int r) {
  RbRow x;
  x.a = s.off[slot * kRbPitch + r];
  x.b = s.off[slot * kRbPitch + r + 1];
  x.valid = (s.bm[slot * 8 + (r >> 5)] >> (r & 31)) & 1u;
  return x;
}

// Closed-form output length of local row r (R5 FirstX cap, R7 NGram count,
// R10 filled null = 1 id, R14 null = empty).
__device__ __forceinline__ int32_t rb_len(const RbF& F, const RbSmem& s, int r) {
  const int kind = F.kind;
  if (kind == 0) {
    const RbRow x = rb_row(s, F.slot[0], r);
    return x.valid ? min(max(x.b - x.a, 0), F.cap[0]) : F.ncap[0];
  }
  if (kind == 1) return F.out_cap;
  long long tot = 0;
  const int k = F.k;
  for (int i = 0; i < k; ++i) {
    const int sl = F.slot[i];
    if (sl < 0) {
      tot += F.cap[i];
      continue;
    }
    const RbRow x = rb_row(s, sl, r);
    tot += x.valid ? min(max(x.b - x.a, 0), F.cap[i]) : F.ncap[i];
  }
  return (int32_t)min(max(tot - (long long)F.n + 1, 0ll), (long long)F.out_cap);
}

__device__ __forceinline__ int32_t rb_len_cached(const RbF& F, const RbSmem& s, int fl, int r) {
  const uint32_t c = s.len[fl * kRbChunk + r];
  return c < kLenBig ? (int32_t)c : rb_len(F, s, r);
}

// Stage the offsets [c0, c0 + nr] and validity words of the group's raw
// columns (cp.async: nothing in flight in registers).
template <class P>
__device__ __forceinline__ void rb_stage(const P& p, const RbSmem& s, const int16_t* cols, int n_cols, int64_t c0,
                                         int nr) {
  const int tid = threadIdx.x;
  const int nw = (nr + 31) >> 5;
  for (int k = 0; k < n_cols; ++k) {
    const int col = cols[k];
    const int32_t* off = p.off[col] + c0;
    int32_t* so = s.off + k * kRbPitch;
    for (int i = tid; i <= nr; i += kRbChunk) cp_async4(so + i, off + i);
    if (tid < nw) {
      const uint32_t* bm = p.svalid[col];
      if (bm != nullptr)
        cp_async4(s.bm + k * 8 + tid, bm + (c0 >> 5) + tid);
      else
        s.bm[k * 8 + tid] = 0xffffffffu;
    }
  }
  cp_async_wait_all();
  __syncthreads();
}

// Lengths of every output of the group for the staged chunk -> s.len, and
// their warp sums -> s.ws (accumulated over chunks when acc).
template <bool kSmall>
__device__ __forceinline__ void rb_lengths(const RbSmem& s, int FL, int nr, bool acc) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const bool in = tid < nr;
  for (int fl = 0; fl < FL; ++fl) {
    const int32_t len = in ? rb_len(s.feat[fl], s, tid) : 0;
    s.len[fl * kRbChunk + tid] = (uint16_t)min((uint32_t)len, kLenBig);
    const long long w = rb_warp_sum<kSmall>(len);
    if (lane == 0) s.ws[fl * 8 + warp] = acc ? s.ws[fl * 8 + warp] + w : w;
  }
}

// ---- id emission ----
__device__ __forceinline__ void rb_store(const Common& c, long long pos, int64_t v) {
  if (pos < c.values_cap)
    c.values[pos] = v;
  else
    atomicExch(c.err, 1);
}

// Canonical stages of q restricted to the bits in `keep` (Clamp -> MapId ->
// SigridHash -> Bucketize order is fixed, so a prefix / suffix split of the
// mask splits the pipeline).
__device__ __forceinline__ void canon_part(const Canon& q, int keep, const int64_t* itab, int64_t& v, bool full) {
  int64_t x[1] = {v};
  canon_apply_nm<1>(q, q.mask & keep, itab, x, 1u, full ? 1u : 0u);
  v = x[0];
}

// Element 0 of a canonical list output's row (valid: the first child id;
// filled null: the fill), loaded one output ahead of its use.
template <class P>
__device__ __forceinline__ int64_t rb_prefetch(const P& p, const RbSmem& s, int fl, int r, bool in) {
  const RbF& F = s.feat[fl];
  if (F.emit != 0) return 0;
  const int sl = F.slot[0];
  const int32_t a = s.off[sl * kRbPitch + r];
  const bool valid = (s.bm[sl * 8 + (r >> 5)] >> (r & 31)) & 1u;
  if (in && valid && s.len[fl * kRbChunk + r] != 0) return __ldg(p.val[F.src0] + a);
  return F.fill;
}

// One element of an NGram source chain (k-th source of program pg) for the
// generic path: element j of the row (start >= 0 valid list, -1 filled null,
// -2 dense bucket).
template <class P>
__device__ __noinline__ int64_t rb_src_elem(const P& p, const SProg& pg, int kk, int32_t start, int64_t row,
                                            int32_t j) {
  const Canon& q = pg.src_cn[kk];
  const Chain& ch = pg.src[kk];
  if (q.ok && start >= -1) {
    int64_t v = start >= 0 ? __ldg(p.val[ch.src] + start + j) : ch.fill;
    canon_part(q, 0xff, p.c.itab, v, start >= 0);
    return v;
  }
  return src_value(p, prog_ops(pg, p.c.ops), pg.tab_off, ch, start, row, j);
}

// Generic list (non-canonical chain) or dense Bucketize output.
template <class P>
__device__ __noinline__ void rb_emit_generic(const P& p, const RbSmem s, const RbF& F, int r, int64_t row,
                                             int32_t len, long long pos) {
  const SProg& pg = p.c.sprogs[F.f];
  const DevOp* ops = prog_ops(pg, p.c.ops);
  if (F.emit == 2) {  // dense Bucketize (R4): one id
    if (len > 0) rb_store(p.c, pos, src_value(p, ops, pg.tab_off, pg.ch, -2, row, 0));
    return;
  }
  const RbRow x = rb_row(s, F.slot[0], r);
  const int32_t start = x.valid ? x.a : -1;
  for (int32_t j = 0; j < len; ++j) rb_store(p.c, pos + j, src_value(p, ops, pg.tab_off, pg.ch, start, row, j));
}

// Canonical chain with its stage set MASK fixed at compile time: Clamp (R6)
// -> MapId (R8) -> SigridHash (R1-R3) -> Bucketize (R4), parameters read
// from the shared-memory record.  A stage runs on a filled null row (full =
// false) only if it follows the FillNull (null_mask, R10).  Element 0 is
// memoised after stage bit memo_after (16: before the first stage).
template <int MASK>
__device__ __forceinline__ int64_t canon_run(const Canon& q, const int64_t* itab, int64_t v, bool full,
                                             int memo_after, long long* memo) {
  const int nmask = q.null_mask;
  if (memo_after == 16) *memo = v;
  if (MASK & CB_CLAMP) {
    if (full || (nmask & CB_CLAMP)) {
      const int64_t lo = q.lo, hi = q.hi;
      v = v < lo ? lo : v;
      v = v > hi ? hi : v;
    }
    if (memo_after == CB_CLAMP) *memo = v;
  }
  if (MASK & CB_MAPID) {
    if (full || (nmask & CB_MAPID)) v = map_lookup(itab, q.map_a, q.map_m, q.map_def, 0, 0, v);
    if (memo_after == CB_MAPID) *memo = v;
  }
  if (MASK & CB_SIGRID) {
    if (full || (nmask & CB_SIGRID)) v = (int64_t)reduce_M(splitmix_H(q.hs ^ (uint64_t)v), q.M);
    if (memo_after == CB_SIGRID) *memo = v;
  }
  if (MASK & CB_BUCKET) {
    if (full || (nmask & CB_BUCKET)) v = upper_bound(itab + q.bk_a, q.bk_m, v);
    if (memo_after == CB_BUCKET) *memo = v;
  }
  return v;
}

// Ids of a canonical list output for this thread's row: element 0 (x0) was
// loaded one output ahead; further elements (multi-id rows) load here.
template <int MASK, class P>
__device__ __forceinline__ void emit_canon(const P& p, const RbSmem& s, const RbF& F, int r, int32_t len,
                                           long long pos, int64_t x0) {
  if (len == 0) return;
  const int sl = F.slot[0];
  const bool valid = (s.bm[sl * 8 + (r >> 5)] >> (r & 31)) & 1u;
  const int ms = F.memo_slot;
  long long* memo = s.memo + max(ms, 0) * kRbChunk + r;  // written only when ms >= 0
  const int ma = ms >= 0 ? F.memo_after : -1;
  rb_store(p.c, pos, canon_run<MASK>(F.cn, p.c.itab, x0, valid, ma, memo));
  if (len > 1) {  // only a valid row holds more than one id
    const int32_t a = s.off[sl * kRbPitch + r];
    const int64_t* vals = p.val[F.src0] + a;
    for (int32_t j = 1; j < len; ++j)
      rb_store(p.c, pos + j, canon_run<MASK>(F.cn, p.c.itab, __ldg(vals + j), true, -1, memo));
  }
}

template <class P>
__device__ __forceinline__ void emit_canon_any(const P& p, const RbSmem& s, const RbF& F, int r, int32_t len,
                                               long long pos, int64_t x0) {
  switch (F.cn.mask & 15) {
    case 0: emit_canon<0>(p, s, F, r, len, pos, x0); break;
    case 1: emit_canon<1>(p, s, F, r, len, pos, x0); break;
    case 2: emit_canon<2>(p, s, F, r, len, pos, x0); break;
    case 3: emit_canon<3>(p, s, F, r, len, pos, x0); break;
    case 4: emit_canon<4>(p, s, F, r, len, pos, x0); break;
    case 5: emit_canon<5>(p, s, F, r, len, pos, x0); break;
    case 6: emit_canon<6>(p, s, F, r, len, pos, x0); break;
    case 7: emit_canon<7>(p, s, F, r, len, pos, x0); break;
    case 8: emit_canon<8>(p, s, F, r, len, pos, x0); break;
    case 9: emit_canon<9>(p, s, F, r, len, pos, x0); break;
    case 10: emit_canon<10>(p, s, F, r, len, pos, x0); break;
    case 11: emit_canon<11>(p, s, F, r, len, pos, x0); break;
    case 12: emit_canon<12>(p, s, F, r, len, pos, x0); break;
    case 13: emit_canon<13>(p, s, F, r, len, pos, x0); break;
    case 14: emit_canon<14>(p, s, F, r, len, pos, x0); break;
    default: emit_canon<15>(p, s, F, r, len, pos, x0); break;
  }
}

// NGram fast path (R7) for a row whose sources each hold at most one id and
// whose providers memoised it earlier in this CTA: the present elements are
// pushed through a WN-register window, a window of n hashes is emitted per
// element from the n-th on.  Returns false (nothing stored) otherwise.
template <int WN, class P>
__device__ __forceinline__ bool ngram_fast(const P& p, const RbSmem& s, const RbF& F, int fl, int pb, int r,
                                           int32_t len, long long pos, uint64_t hs0, int64_t M) {
  const int n = F.n, K = F.k;
  bool ok = true;
  for (int kk = 0; kk < K; ++kk) {
    const int pv = F.prov[kk];
    const int sl = F.slot[kk];
    if (pv < pb || pv >= pb + fl || sl < 0) return false;
    const RbRow x = rb_row(s, sl, r);
    const int32_t lk = x.valid ? min(max(x.b - x.a, 0), F.cap[kk]) : F.ncap[kk];
    ok &= lk <= 1 && (lk == 0 || s.len[(pv - pb) * kRbChunk + r] >= 1);
  }
  if (!ok) return false;
  uint64_t w[WN];
#pragma unroll
  for (int i = 0; i < WN; ++i) w[i] = 0;
  int32_t cnt = 0;
  for (int kk = 0; kk < K; ++kk) {
    const int sl = F.slot[kk];
    const RbRow x = rb_row(s, sl, r);
    const int32_t lk = x.valid ? min(max(x.b - x.a, 0), F.cap[kk]) : F.ncap[kk];
    if (lk == 0) continue;
    const uint64_t e = (uint64_t)s.memo[F.pslot[kk] * kRbChunk + r];
#pragma unroll
    for (int i = 0; i < WN - 1; ++i) w[i] = w[i + 1];
    w[WN - 1] = e;
    ++cnt;
    if (cnt >= n && cnt - n < len) {
      uint64_t h = hs0;
#pragma unroll
      for (int i = 0; i < WN; ++i)
        if (i >= WN - n) h = splitmix_H(h ^ w[i]);
      int64_t v = (int64_t)reduce_M(h, M);
      if (F.cn.mask) canon_part(F.cn, 0xff, p.c.itab, v, true);
      rb_store(p.c, pos + (cnt - n), v);
    }
  }
  return true;
}

// NGram (R7): c = concatenation of the k source lists; window j hashes
// c[j .. j+n) into H(salt) in order; the post ops run on reduce(h, M).
// A source whose provider ran earlier in this CTA reads its memoised
// element 0 (rows with at most one id); anything else is recomputed.
template <class P>
__device__ __noinline__ void rb_emit_ngram(const P& p, const RbSmem s, const RbF& F, int fl, int r, int64_t row,
                                           int32_t len, long long pos, int pb) {
  const SProg& pg = p.c.sprogs[F.f];
  const int n = F.n, K = F.k;
  const uint64_t hs0 = pg.ng.hsalt;
  const int64_t M = pg.ng.M;
  uint64_t w[kMaxNgramK];  // the last n elements, w[kMaxNgramK - 1] newest
#pragma unroll
  for (int i = 0; i < kMaxNgramK; ++i) w[i] = 0;
  int32_t cnt = 0;
  for (int kk = 0; kk < K && cnt - n + 1 < len; ++kk) {
    const int sl = F.slot[kk];
    int32_t lk, start;
    if (sl < 0) {
      lk = F.cap[kk];
      start = -2;
    } else {
      const RbRow x = rb_row(s, sl, r);
      lk = x.valid ? min(max(x.b - x.a, 0), F.cap[kk]) : F.ncap[kk];
      start = x.valid ? x.a : -1;
    }
    const int pv = F.prov[kk];
    const bool memo = pv >= pb && pv < pb + fl && lk <= 1 && (lk == 0 || s.len[(pv - pb) * kRbChunk + r] >= 1);
    const int ps = memo ? F.pslot[kk] : 0;
    for (int32_t j = 0; j < lk && cnt - n + 1 < len; ++j) {
      const int64_t e = memo ? s.memo[ps * kRbChunk + r] : rb_src_elem(p, pg, kk, start, row, j);
#pragma unroll
      for (int i = 0; i < kMaxNgramK - 1; ++i) w[i] = w[i + 1];
      w[kMaxNgramK - 1] = (uint64_t)e;
      ++cnt;
      if (cnt >= n) {
        uint64_t h = hs0;
#pragma unroll
        for (int i = 0; i < kMaxNgramK; ++i)
          if (i >= kMaxNgramK - n) h = splitmix_H(h ^ w[i]);
        int64_t v = (int64_t)reduce_M(h, M);
        if (F.cn.ok)
          canon_part(F.cn, 0xff, p.c.itab, v, true);
        else
          v = apply_id_ops(prog_ops(pg, p.c.ops), p.c.itab, pg.tab_off, v, pg.ch.op_begin, pg.ch.op_end);
        rb_store(p.c, pos + (cnt - n), v);
      }
    }
  }
}

#ifndef RAP_RB_MIN_CTAS
#define RAP_RB_MIN_CTAS 2
#endif
template <int MD, int MS, bool kSmall>
__global__ void __launch_bounds__(kRbChunk, RAP_RB_MIN_CTAS) rap_rows_kernel(const __grid_constant__ RbParams<MD, MS> p) {
  unsigned char* const smem = rap_dyn_smem;
  __shared__ CtaState cs;
  __shared__ int16_t s_slot[MS];  // raw sparse column -> staged slot (-1: not staged)
  __shared__ int16_t s_cols[MS];  // staged slot -> raw sparse column
  __shared__ unsigned long long s_mask[(MS + 63) / 64];
  __shared__ int s_last, s_fmax;
  const RbGeom& g = p.g;
  const Common& c = p.c;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int F = c.n_sparse_out;
  const RbSmem s = rb_carve(smem, g, F);
  const int n_rb = g.n_rb;
  const int grp = (int)blockIdx.x / n_rb, rb = (int)blockIdx.x - grp * n_rb;
  const int pb = g.fg_off[grp], pe = g.fg_off[grp + 1];  // processing indices of my group
  const int FL = pe - pb;
  const int64_t B = c.n_rows;
  const int64_t R0 = (int64_t)rb * g.rows_rb;
  const int64_t R1 = min(B, R0 + (int64_t)g.rows_rb);
  const int nrows = (int)max((int64_t)0, R1 - R0);
  const int nch = (nrows + kRbChunk - 1) / kRbChunk;
  const long long chain0 = c.chain ? (long long)__ldg(c.offsets) : 0ll;
  unsigned long long* const pub = g.sched + 2;  // CTAs whose totals are stored
  trace_stamp(c, 0);

  if (tid == 0) {
    mbar_init(&cs.bar, 1);
    cs.phase = 0;
    cs.dgroup = -1;
    s_fmax = 0;
    if (blockIdx.x == 0 && F == 0 && !c.chain && c.offsets) c.offsets[0] = 0;  // no sparse outputs (R17)
  }
  for (int i = tid; i < (MS + 63) / 64; i += kRbChunk) s_mask[i] = 0ull;
  __syncthreads();
  // the group's output records -> shared memory; the raw columns they read
  if (tid < FL) {
    const int f = __ldg(g.perm + pb + tid);
    const RbFeat& G = g.feat[f];
    RbF& R = s.feat[tid];
    R.kind = __ldg(&G.kind);
    R.emit = __ldg(&G.emit);
    R.n = __ldg(&G.n);
    R.k = __ldg(&G.k);
    R.out_cap = __ldg(&G.out_cap);
    R.memo_slot = __ldg(&G.memo_slot);
    R.memo_mask = __ldg(&G.memo_mask);
    R.f = f;
    const int kk = R.kind == 1 ? 0 : R.k;
    for (int i = 0; i < kMaxNgramK; ++i) {
      R.cap[i] = __ldg(&G.cap[i]);
      R.ncap[i] = __ldg(&G.ncap[i]);
      const int src = __ldg(&G.src[i]);
      R.slot[i] = (int16_t)src;  // raw column for now, slot below
      if (i < kk && src >= 0) atomicOr(&s_mask[src >> 6], 1ull << (src & 63));
    }
    for (int i = 0; i < kMaxNgramK; ++i) {
      R.prov[i] = (int16_t)__ldg(&G.prov[i]);
      R.pslot[i] = (int16_t)__ldg(&G.pslot[i]);
    }
    const SProg& pg = c.sprogs[f];
    R.src0 = __ldg(&G.src[0]);
    R.fill = pg.ch.fill;
    R.cn = pg.cn;
    {  // memo point: after the last stage of the provider prefix present in the chain
      const int pm = R.memo_mask & R.cn.mask;
      int ma = pm ? 1 : 16;
      while (pm >> 1 >= ma) ma <<= 1;
      R.memo_after = R.memo_slot >= 0 ? ma : -1;
    }
    atomicMax(&s_fmax, f);
  }
  __syncthreads();
  int n_cols = 0;
  for (int i = 0; i < (MS + 63) / 64; ++i) n_cols += __popcll(s_mask[i]);
  for (int col = tid; col < MS; col += kRbChunk) {
    const unsigned long long m = s_mask[col >> 6];
    int before = __popcll(m & ((1ull << (col & 63)) - 1ull));
    for (int i = 0; i < (col >> 6); ++i) before += __popcll(s_mask[i]);
    const bool on = (m >> (col & 63)) & 1ull;
    s_slot[col] = on ? (int16_t)before : (int16_t)-1;
    if (on) s_cols[before] = (int16_t)col;
  }
  __syncthreads();
  if (tid < FL) {
    RbF& R = s.feat[tid];
    const int kk = R.kind == 1 ? 0 : R.k;
    for (int i = 0; i < kMaxNgramK; ++i) R.slot[i] = (i < kk && R.slot[i] >= 0) ? s_slot[R.slot[i]] : (int16_t)-1;
  }
  __syncthreads();

  // (1) per-output totals of my rows -> agg, then announce the CTA
  for (int ch = 0; ch < nch; ++ch) {
    const int64_t c0 = R0 + (int64_t)ch * kRbChunk;
    const int nr = (int)min((int64_t)kRbChunk, R1 - c0);
    rb_stage(p, s, s_cols, n_cols, c0, nr);
    rb_lengths<kSmall>(s, FL, nr, ch > 0);
    __syncthreads();
  }
  if (tid < FL) {
    long long tot = 0;
    if (nch > 0)
#pragma unroll
      for (int w = 0; w < 8; ++w) tot += s.ws[tid * 8 + w];
    g.agg[(int64_t)s.feat[tid].f * n_rb + rb] = (unsigned long long)tot;
  }
  __syncthreads();
  if (tid == 0) {
    __threadfence();  // release: the block's totals before the announcement
    atomicAdd(pub, 1ull);
  }
  trace_stamp(c, 1);

  // (2) dense blocks, round robin over the CTAs (independent of the scan)
  for (int64_t d = blockIdx.x; d < c.n_dense_tiles; d += gridDim.x) {
    const uint32_t gi = (uint32_t)d % (uint32_t)c.n_groups;
    dense_block(p, (int)gi, (int64_t)((uint32_t)d / (uint32_t)c.n_groups), 0, cs);
    __syncthreads();
  }
  trace_stamp(c, 2);

  if (FL > 0 && nrows > 0) {
    // (3) wait until every CTA announced its totals (all resident: cooperative launch)
    if (tid == 0) {
      int ns = 32;
      while (ld_acquire(pub) < (unsigned long long)gridDim.x) {
        __nanosleep(ns);
        ns = min(ns * 2, 256);
      }
    }
    __syncthreads();
    trace_stamp(c, 3);
    // T[f] = sum over all row blocks, L[f] = sum over row blocks below mine,
    // for f = 0 .. fmax (output order); warp w reduces outputs w, w + 8, ...
    const int fmax = s_fmax;
    long long* sT = reinterpret_cast<long long*>(s.dense);
    long long* sL = sT + (fmax + 1);
    for (int f = warp; f <= fmax; f += kWarps) {
      const unsigned long long* row = g.agg + (int64_t)f * n_rb;
      long long t = 0, l = 0;
#pragma unroll 4
      for (int j = lane; j < n_rb; j += 32) {
        const long long v = ld_cg64(row + j);
        t += v;
        l += j < rb ? v : 0;
      }
      t = rb_warp_sum<kSmall>(t);
      l = rb_warp_sum<kSmall>(l);
      if (lane == 0) {
        sT[f] = t;
        sL[f] = l;
      }
    }
    __syncthreads();
    if (tid == 0) {  // exclusive prefix over outputs in feature-major order
      long long P = chain0;
      for (int f = 0; f <= fmax; ++f) {
        const long long t = sT[f];
        sT[f] = P;
        P += t;
      }
    }
    __syncthreads();
    if (tid < FL) {
      const int f = s.feat[tid].f;
      s.base[tid] = sT[f] + sL[f];
    }
    __syncthreads();
    trace_stamp(c, 4);

    // (4) lengths, offsets and ids, chunk by chunk
    for (int ch = 0; ch < nch; ++ch) {
      const int64_t c0 = R0 + (int64_t)ch * kRbChunk;
      const int nr = (int)min((int64_t)kRbChunk, R1 - c0);
      if (nch > 1) {
        rb_stage(p, s, s_cols, n_cols, c0, nr);
        rb_lengths<kSmall>(s, FL, nr, false);
        __syncthreads();
      }
      if (tid < FL) {  // warp bases of this chunk; the running base advances
        long long b = s.base[tid];
#pragma unroll
        for (int w = 0; w < 8; ++w) {
          s.wb[tid * 8 + w] = b;
          b += s.ws[tid * 8 + w];
        }
        s.base[tid] = b;
      }
      __syncthreads();
      const bool in = tid < nr;
      const int64_t row = c0 + tid;
      int64_t nx = rb_prefetch(p, s, 0, tid, in);
      for (int fl = 0; fl < FL; ++fl) {
        const int64_t x0 = nx;
        if (fl + 1 < FL) nx = rb_prefetch(p, s, fl + 1, tid, in);
        const RbF& Fd = s.feat[fl];
        const int32_t len = in ? rb_len_cached(Fd, s, fl, tid) : 0;
        const long long pos = s.wb[fl * 8 + warp] + rb_warp_excl<kSmall>(len, lane);
        if (!in) continue;
        const int f = Fd.f;
        const int64_t oi = (int64_t)f * B + row;
        c.lengths[oi] = len;
        c.offsets[oi] = pos;
        if (f == F - 1 && row == B - 1) c.offsets[(int64_t)F * B] = pos + len;
        const int emit = Fd.emit;
        if (emit == 0) {  // canonical list: Clamp -> MapId -> SigridHash -> Bucketize subset
          emit_canon_any(p, s, Fd, tid, len, pos, x0);
        } else if (emit == 3) {
          if (len > 0) {
            const SProg& pg = c.sprogs[f];
            const uint64_t hs0 = pg.ng.hsalt;
            const int64_t M = pg.ng.M;
            const bool done = Fd.n <= 4 ? ngram_fast<4>(p, s, Fd, fl, pb, tid, len, pos, hs0, M)
                                        : ngram_fast<8>(p, s, Fd, fl, pb, tid, len, pos, hs0, M);
            if (!done) rb_emit_ngram(p, s, Fd, fl, tid, row, len, pos, pb);
          }
        } else {
          rb_emit_generic(p, s, Fd, tid, row, len, pos);
        }
      }
      __syncthreads();
    }
  }
  trace_stamp(c, 5);

  // last CTA out: reset the counters (launch parameters stay the same)
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    const unsigned long long prev = atomicAdd(g.sched, 1ull);
    s_last = (prev == (unsigned long long)gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  if (s_last && tid == 0) {
    __threadfence();
    g.sched[0] = 0ull;
    g.sched[2] = 0ull;
    __threadfence();
  }
}

template <int MD, int MS, bool kSmall>
static int launch_rows_t(const Common& c, const RbGeom& g, const LaunchRaw& raw, int smem, cudaStream_t st) {
  static_assert(sizeof(RbParams<MD, MS>) <= 32000, "kernel parameter block too large");
  // the attribute is set on every launch whose smem differs from the value
  // last set on this device (plans with different geometries alternate)
  static thread_local int last_dev = -1, last_smem = -1;
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev != last_dev || smem != last_smem) {
    cudaError_t e = cudaFuncSetAttribute(rap_rows_kernel<MD, MS, kSmall>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         smem);
    if (e != cudaSuccess) return (int)e;
    last_dev = dev;
    last_smem = smem;
  }
  RbParams<MD, MS> p;
  memset(&p, 0, sizeof(p));
  p.c = c;
  p.g = g;
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
  cfg.gridDim = dim3((unsigned)(g.n_rb * g.n_fg));
  cfg.blockDim = dim3(kRbChunk);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;  // every CTA resident: (3) waits on all of them
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, rap_rows_kernel<MD, MS, kSmall>, p);
  if (e != cudaSuccess) return (int)e;
  return (int)cudaGetLastError();
}

int launch_rows(const Common& c, const RbGeom& g, const LaunchRaw& raw, int smem_bytes, void* stream) {
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (raw.n_dense > kRbMaxDense || raw.n_sparse > kRbMaxCols) return (int)cudaErrorInvalidValue;
  if (g.small) return launch_rows_t<kRbMaxDense, kRbMaxCols, true>(c, g, raw, smem_bytes, st);
  return launch_rows_t<kRbMaxDense, kRbMaxCols, false>(c, g, raw, smem_bytes, st);
}

int rows_dense_bytes(int max_width) {
  const int tile = kDenseBlockRows * (max_width | 1) * 4;
  return kDProgBytes + dense_in_bytes() + align_up(tile, 16);
}

int rows_smem_bytes(int dense_bytes, int max_fl, int max_cols, int n_memo, int n_sparse_out) {
  int o = rb_region0(dense_bytes, n_memo, n_sparse_out);
  o += 2 * rb_align(max_fl * 8 * 8);
  o += rb_align(max_fl * 8);
  o += rb_align(max_fl * (int)sizeof(RbF));
  o += rb_align(max_cols * kRbPitch * 4);
  o += rb_align(max_cols * 8 * 4);
  o += rb_align(max_fl * kRbChunk * 2);
  return o;
}

int rows_occupancy(int smem_bytes, int* ctas_per_sm) {
  cudaError_t e = cudaFuncSetAttribute(rap_rows_kernel<kRbMaxDense, kRbMaxCols, true>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(rap_rows_kernel<kRbMaxDense, kRbMaxCols, false>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
  if (e == cudaSuccess)
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, rap_rows_kernel<kRbMaxDense, kRbMaxCols, true>,
                                                      kRbChunk, smem_bytes);
  return (int)e;
}

}  // namespace rapk
