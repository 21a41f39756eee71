// rap_rows_skel.cuh — skeleton of the row-block fused kernel (sm_100a),
// shared by the built-in interpreter (rap_rows.cu) and the plan-specialised
// kernel generated at plan time (rap_jit.cpp).
//
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
#pragma once
#ifndef RAP_BASES_UNROLL
#define RAP_BASES_UNROLL 4
#endif
#ifndef __CUDACC_RTC__
#include <cuda_runtime.h>
#include <stdint.h>
#endif

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
  long long* ide0;       // [id_slots] values index of ids[slot][0] (kRbIdNone: not staged)
  long long* ids;        // [id_slots][kRbIdCap] the chunk's ids of the slot's column
  int pitch;             // staged offsets per column (g.pitch, default kRbPitch)
  unsigned char* tabs;   // generated kernel: [mbarrier, 16 B][tables staged at launch] (the layout's end)
};

constexpr long long kRbIdNone = -(1ll << 61);  // ide0 of a column whose chunk ids were not staged

__host__ __device__ inline int rb_align(int x) { return (x + 15) & ~15; }

__host__ __device__ inline int rb_region0(int dense_bytes, int n_memo, int max_f) {
  const int m = n_memo * kRbChunk * 8, r = 2 * (max_f + 1) * 8;  // phase (3): T[f], L[f]
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
  if (g.feat_recs) o += rb_align(g.max_fl * (int)sizeof(RbF));
  s.pitch = g.pitch > 0 ? g.pitch : kRbPitch;
  s.off = reinterpret_cast<int32_t*>(smem + o);
  o += rb_align(g.max_cols * s.pitch * 4);
  s.bm = reinterpret_cast<uint32_t*>(smem + o);
  o += rb_align(g.max_cols * 8 * 4);
  s.len = g.len_cache ? reinterpret_cast<uint16_t*>(smem + o) : nullptr;
  if (g.len_cache) o += rb_align(g.max_fl * kRbChunk * 2);
  s.ide0 = reinterpret_cast<long long*>(smem + o);
  o += rb_align(g.id_slots * 8);
  s.ids = reinterpret_cast<long long*>(smem + o);
  o += g.id_slots * kRbIdCap * 8;
  s.tabs = smem + rb_align(o);
  return s;
}

__device__ __forceinline__ ulonglong2 ld_cg128(const ulonglong2* p) {
  ulonglong2 v;
  asm volatile("ld.global.cg.v2.u64 {%0, %1}, [%2];" : "=l"(v.x), "=l"(v.y) : "l"(p));
  return v;
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

// Exclusive warp scan of 0/1 flags (rows holding at most one id).
__device__ __forceinline__ long long rb_ballot_excl(bool f, int lane) {
  return (long long)__popc(__ballot_sync(0xffffffffu, f) & ((1u << lane) - 1u));
}

// ---- staged raw rows ----
struct RbRow {
  int32_t a, b;
  bool valid;
};

__device__ __forceinline__ RbRow rb_row(const RbSmem& s, int slot, int r) {
  RbRow x;
  x.a = s.off[slot * s.pitch + r];
  x.b = s.off[slot * s.pitch + r + 1];
  x.valid = (s.bm[slot * 8 + (r >> 5)] >> (r & 31)) & 1u;
  return x;
}
// Same with the pitch a compile-time constant (generated code).
template <int PITCH>
__device__ __forceinline__ RbRow rb_row_p(const RbSmem& s, int slot, int r) {
  RbRow x;
  x.a = s.off[slot * PITCH + r];
  x.b = s.off[slot * PITCH + r + 1];
  x.valid = (s.bm[slot * 8 + (r >> 5)] >> (r & 31)) & 1u;
  return x;
}

// Barrier of the threads that run the sparse phases: every thread, or (the
// generated kernel with a dense warp) warps 0-6 on named barrier 1.
template <bool kDW>
__device__ __forceinline__ void rb_sync() {
  if (kDW)
    asm volatile("bar.sync 1, 224;" ::: "memory");
  else
    __syncthreads();
}

// Stage the ids val[a0, a1) of one column's chunk into dst (kRbIdCap slots):
// dst[j] = val[e0 + j] with e0 = a0 - h (h = 1 when val + a0 is not 16-byte
// aligned, so the bulk copy's source and destination are), the 16-byte
// aligned body by one bulk copy onto ibar, the <= 2 unaligned end ids by plain
// loads (never a byte outside [a0, a1)).  Ranges that do not fit (long lists)
// are not staged (e0 = kRbIdNone: the emitter reads them from global).
__device__ __forceinline__ void rb_stage_ids(const int64_t* val, int32_t a0, int32_t a1, long long* dst,
                                             long long* e0, uint64_t* ibar) {
  const int n = a1 - a0;
  const int h = (reinterpret_cast<uintptr_t>(val + a0) & 15) ? 1 : 0;
  if (val == nullptr || n < 0 || n + h > kRbIdCap) {
    *e0 = kRbIdNone;
    mbar_arrive_expect(ibar, 0u);
    return;
  }
  const int t = (n > h && (reinterpret_cast<uintptr_t>(val + a1) & 15)) ? 1 : 0;
  const int nb = n - h - t;  // body ids (16-byte aligned at both ends)
  mbar_arrive_expect(ibar, nb > 0 ? (uint32_t)nb * 8u : 0u);
  if (nb > 0) bulk_g2s(dst + 2 * h, val + a0 + h, (uint32_t)nb * 8u, ibar);
  if (h && n > 0) dst[1] = __ldg(val + a0);
  if (t) dst[n - 1 + h] = __ldg(val + a1 - 1);
  *e0 = (long long)a0 - h;
}

// Stage the offsets [c0, c0 + nr] and validity words of the group's raw
// columns: thread 0 issues one bulk copy (TMA engine, cp.async.bulk) per
// column body onto the CTA's staging mbarrier; warp 0 loads the <= 3
// unaligned tail words (and whole columns whose base is not 16-byte aligned).
template <bool kDW, class P>
__device__ __forceinline__ void rb_stage(const P& p, const RbSmem& s, const int16_t* cols, int n_cols, int64_t c0,
                                         int nr, uint64_t* bar, int* phase, int n_ids = 0, uint64_t* ibar = nullptr) {
  // thread k < n_cols stages column k: one bulk copy (TMA engine) each for the
  // 16-byte-aligned body of its offsets and validity words, arriving on the
  // staging mbarrier (expected arrivals = n_cols) with those bytes; the <= 3
  // unaligned tail words (or a whole misaligned column) by plain loads
  const int tid = threadIdx.x;
  const int no = nr + 1, nw = (nr + 31) >> 5;
  if (n_cols == 0) return;  // the group reads no list column
  if (tid == 0) fence_proxy_async();  // the previous chunk's generic reads of the staging area come first
  rb_sync<kDW>();
  if (tid < n_cols) {
    const int k = tid, col = cols[k];
    const int32_t* src = p.off[col] + c0;
    // slots < n_ids: the chunk's id range [off[c0], off[c0 + nr]) too (its
    // two bounds are loaded beside the offsets' bulk copy)
    int32_t a0 = 0, a1 = 0;
    if (k < n_ids) {
      a0 = __ldg(src);
      a1 = __ldg(src + nr);
    }
    const bool oa = (reinterpret_cast<uintptr_t>(src) & 15) == 0;
    const uint32_t ob = oa ? ((uint32_t)(no * 4) & ~15u) : 0u;
    const uint32_t* bm = p.svalid[col];
    const uint32_t* bs = bm ? bm + (c0 >> 5) : nullptr;
    const bool wa = bs != nullptr && (reinterpret_cast<uintptr_t>(bs) & 15) == 0;
    const uint32_t wb = wa ? ((uint32_t)(nw * 4) & ~15u) : 0u;
    mbar_arrive_expect(bar, ob + wb);
    if (ob) bulk_g2s(s.off + k * s.pitch, src, ob, bar);
    if (wb) bulk_g2s(s.bm + k * 8, bs, wb, bar);
    if (k < n_ids) rb_stage_ids(p.val[col], a0, a1, s.ids + k * kRbIdCap, s.ide0 + k, ibar);
#ifdef RAP_PREFETCH_IDS
    // the chunk's ids, read only in the emit phase, prefetched into L2 now
    // (one bulk prefetch of the whole 16-byte units inside the range)
    if (k >= n_ids) {
      const int32_t b0 = __ldg(src), b1 = __ldg(src + nr);
      const uintptr_t lo = (reinterpret_cast<uintptr_t>(p.val[col] + b0) + 15) & ~(uintptr_t)15;
      const uintptr_t hi = reinterpret_cast<uintptr_t>(p.val[col] + b1) & ~(uintptr_t)15;
      if (b1 > b0 && hi > lo)
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(lo), "r"((uint32_t)(hi - lo)) : "memory");
    }
#endif
  }
  // the words outside the bulk copies (an unaligned offsets tail, validity
  // words of an unaligned bitmap: 3 of 4 row blocks of 224 rows), 8 threads
  // per column so their loads are in flight together
  {
    const int nthr = kDW ? 224 : (int)blockDim.x;
    for (int t = tid; t < n_cols * 8; t += nthr) {
      const int k = t >> 3, j = t & 7, col = cols[k];
      const int32_t* src = p.off[col] + c0;
      const uint32_t ob = (reinterpret_cast<uintptr_t>(src) & 15) == 0 ? ((uint32_t)(no * 4) & ~15u) : 0u;
      for (int i = (int)(ob / 4) + j; i < no; i += 8) s.off[k * s.pitch + i] = __ldg(src + i);
      if (j < nw) {
        const uint32_t* bm = p.svalid[col];
        if (bm == nullptr) {
          s.bm[k * 8 + j] = 0xffffffffu;
        } else {
          const uint32_t* bs = bm + (c0 >> 5);
          const uint32_t wb = (reinterpret_cast<uintptr_t>(bs) & 15) == 0 ? ((uint32_t)(nw * 4) & ~15u) : 0u;
          if (j >= (int)(wb / 4)) s.bm[k * 8 + j] = __ldg(bs + j);
        }
      }
    }
  }
  mbar_wait(bar, (uint32_t)*phase);
  rb_sync<kDW>();
  if (tid == 0) *phase ^= 1;
}

// ---- id emission ----
// Output stores.  The outputs are write-only in the kernel, so the stores are
// emitted as st.global without a memory clobber: the compiler may move shared
// loads of later outputs above them (a store through a plain generic pointer
// could alias shared memory and would pin every later LDS behind it).
// The generated kernel stores its outputs with the streaming hint (st.global.cs,
// evict-first in L2): C2 on B200 with inputs and outputs rotating through HBM,
// 55.8 -> 47.6 us per launch -- written-once output lines no longer push
// the plan's tables and the next lines' staging out of L2.
#ifdef RAP_ST_CS
#define RAP_STG "st.global.cs"
#else
#define RAP_STG "st.global"
#endif
// Raw inputs read once (ids, dense values): streaming loads when RAP_LD_CS.
template <class T>
__device__ __forceinline__ T rap_ldin(const T* p) {
#ifdef RAP_LD_CS
  return __ldcs(p);
#else
  return __ldg(p);
#endif
}
__device__ __forceinline__ int64_t rap_ldin(const int64_t* p) {
#ifdef RAP_LD_CS
  return (int64_t)__ldcs(reinterpret_cast<const long long*>(p));
#else
  return (int64_t)__ldg(reinterpret_cast<const long long*>(p));
#endif
}
__device__ __forceinline__ void stg_s32(int32_t* p, int32_t v) {
  asm volatile(RAP_STG ".s32 [%0], %1;" ::"l"(p), "r"(v));
}
__device__ __forceinline__ void stg_s64(int64_t* p, int64_t v) {
  asm volatile(RAP_STG ".s64 [%0], %1;" ::"l"(p), "l"(v));
}
// Predicated forms (one instruction, no branch around it).  RAP_ST_PLAIN:
// through the st.global.cs intrinsic instead of volatile asm, so the compiler
// may move them and the loads of later outputs past each other.
#ifdef RAP_ST_PLAIN
__device__ __forceinline__ void stg_s32_if(bool q, int32_t* p, int32_t v) {
  if (q) __stcs(p, v);
}
__device__ __forceinline__ void stg_s64_if(bool q, int64_t* p, int64_t v) {
  if (q) __stcs(reinterpret_cast<long long*>(p), (long long)v);
}
#else
__device__ __forceinline__ void stg_s32_if(bool q, int32_t* p, int32_t v) {
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q " RAP_STG ".s32 [%0], %1;\n\t}" ::"l"(p), "r"(v),
               "r"((unsigned)q));
}
__device__ __forceinline__ void stg_s64_if(bool q, int64_t* p, int64_t v) {
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q " RAP_STG ".s64 [%0], %1;\n\t}" ::"l"(p), "l"(v),
               "r"((unsigned)q));
}
#endif
// A value store of element pos (R17 values) in the launch's value type:
// int64, or int32 under Cast (RAP_OUT_VALUES_I32; the generated kernel
// compiles one variant per type, RAP_VALUES_I32 / RAP_VALUES_I64).
__device__ __forceinline__ bool values_i32(const Common& c) {
#if defined(RAP_VALUES_I32)
  return true;
#elif defined(RAP_VALUES_I64)
  return false;
#else
  return c.vi32 != 0;
#endif
}
__device__ __forceinline__ void stv_if(bool q, const Common& c, long long pos, int64_t v) {
  if (values_i32(c))
    stg_s32_if(q, reinterpret_cast<int32_t*>(c.values) + pos, (int32_t)v);
  else
    stg_s64_if(q, c.values + pos, v);
}
__device__ __forceinline__ void rb_store(const Common& c, long long pos, int64_t v) {
  if (pos < c.values_cap) {
    if (values_i32(c))
      stg_s32(reinterpret_cast<int32_t*>(c.values) + pos, (int32_t)v);
    else
      stg_s64(c.values + pos, v);
  } else {
    atomicExch(c.err, 1);
  }
}
// lengths[oi] and offsets[oi] of one (output, row)
__device__ __forceinline__ void rb_store_lo(const Common& c, int64_t oi, int32_t len, long long pos) {
  stg_s32(c.lengths + oi, len);
  stg_s64(c.offsets + oi, pos);
}

// Canonical stages of q restricted to the bits in `keep` (Clamp -> MapId ->
// SigridHash -> Bucketize order is fixed, so a prefix / suffix split of the
// mask splits the pipeline).
__device__ __forceinline__ void canon_part(const Canon& q, int keep, const int64_t* itab, int64_t& v, bool full) {
  int64_t x[1] = {v};
  canon_apply_nm<1>(q, q.mask & keep, itab, x, 1u, full ? 1u : 0u);
  v = x[0];
}


// Raw dense value of a row with the R14 null rule (cleared validity bit ->
// NaN), for generated dense code.
template <class P>
__device__ __forceinline__ float rb_dense_in(const P& p, int col, int64_t row) {
  const uint32_t* bm = p.dvalid[col];
  const float v = rap_ldin(p.dense[col] + row);
  if (bm == nullptr) return v;
  return ((__ldg(bm + (row >> 5)) >> (row & 31)) & 1u) ? v : __int_as_float(0x7fc00000);
}

// Store rows [0, nr) of a row-major tile (pitch floats per row, the first
// width = d_out columns) to dense_out rows [d0, d0 + nr).
__device__ __forceinline__ void rb_tile_store(const Common& c, const float* tile, int pitch, int width, int64_t d0,
                                              int nr) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  float* out = c.dense_out + d0 * c.ld;
  if (c.ld == width && pitch == width) {
    const int n = nr * width;  // one contiguous run
    if ((reinterpret_cast<uintptr_t>(out) & 15) == 0 && (n & 3) == 0) {
      float4* o4 = reinterpret_cast<float4*>(out);
      const float4* t4 = reinterpret_cast<const float4*>(tile);
      for (int i = tid; i < (n >> 2); i += kRbChunk) o4[i] = t4[i];
    } else {
      for (int i = tid; i < n; i += kRbChunk) out[i] = tile[i];
    }
  } else {
    for (int r = warp; r < nr; r += kWarps)
      for (int cc = lane; cc < width; cc += 32) out[r * c.ld + cc] = tile[r * pitch + cc];
  }
}

// One warp stores rows [0, nr) of a row-major tile (pitch floats per row,
// the first width = d_out columns) to dense_out rows [d0, d0 + nr).
__device__ __forceinline__ void rb_tile_store_warp(const Common& c, const float* tile, int pitch, int width,
                                                   int64_t d0, int nr) {
  const int lane = threadIdx.x & 31;
  float* out = c.dense_out + d0 * c.ld;
  if (c.ld == width && pitch == width) {
    const int n = nr * width;
    if ((reinterpret_cast<uintptr_t>(out) & 15) == 0 && (n & 3) == 0) {
      float4* o4 = reinterpret_cast<float4*>(out);
      const float4* t4 = reinterpret_cast<const float4*>(tile);
      for (int i = lane; i < (n >> 2); i += 32) __stcs(o4 + i, t4[i]);
    } else {
      for (int i = lane; i < n; i += 32) __stcs(out + i, tile[i]);
    }
  } else {
    for (int r = 0; r < nr; ++r)
      for (int cc = lane; cc < width; cc += 32) __stcs(out + r * c.ld + cc, tile[r * pitch + cc]);
  }
}

// ---- loop emitter of the generated kernel (rap_jit.cpp emit_loop) ----
// The plan's outputs become rows of __constant__ tables and the emit phase
// loops over them (NGram units: k providers + their NGram per iteration; then
// the single canonical outputs), so the code a warp streams is a few short
// loop bodies instead of one straight-line block per output.
struct JLCanon {  // a canonical output holding at most one id per row (FirstX <= 1)
  long long fill, lo, hi, map_def, map_a, bk_a, M;
  unsigned long long hs;
  int slot, col, f, q;           // staged slot, raw column, output index, processing index
  int cap, ncap, flags, nullm;   // flags: CB_* stages of the chain; nullm: stages that apply to filled nulls
  int map_m, bk_m, bk_row, memo; // bk_row: row of the level-0 / sample tables; memo: stage bit after which the
                                 // NGram word is taken (16: before any stage, 0: none)
  int last, pad;                 // last: f == F - 1 (writes offsets[F * B])
};
template <int K>
struct JLNgram {
  unsigned long long hsalt;
  long long M;
  int f, q, out_cap, last;
  int slot[K], cap[K], ncap[K];
};

// One canonical output of the loop emitter: lengths, offsets, the value of
// element 0 (the chain on the prefetched first id) and its NGram word.
template <bool kSmall, class P>
__device__ __forceinline__ void jl_canon(const P& p, const RbSmem& s, const JLCanon& Q, const long long* l0,
                                         const int64_t* const* smp, int r, int wi, int lane, bool in, int64_t row,
                                         int64_t B, int64_t pf, int64_t* memo, int32_t* len, bool& ovf) {
  const Common& c = p.c;
  const RbRow X = rb_row_p<kRbPitch>(s, Q.slot, r);
  const int32_t L = in ? (X.valid ? min(max(X.b - X.a, 0), Q.cap) : Q.ncap) : 0;
  *len = L;
  const long long P0 = s.wb[Q.q * 8 + wi] + rb_ballot_excl(L != 0, lane);
  stg_s32_if(in, c.lengths + ((int64_t)Q.f * B + row), L);
  stg_s64_if(in, c.offsets + ((int64_t)Q.f * B + row), P0);
  if (Q.last) stg_s64_if(in && row == B - 1, c.offsets + (int64_t)(Q.f + 1) * B, P0 + L);
  ovf |= P0 + L > c.values_cap;
  const bool valid = X.valid;
  int64_t v = valid ? pf : Q.fill;
  if (Q.memo == 16) *memo = v;
  if (Q.flags & CB_CLAMP) {
    const int64_t t = v < Q.lo ? Q.lo : (v > Q.hi ? Q.hi : v);
    v = (valid || (Q.nullm & CB_CLAMP)) ? t : v;
    if (Q.memo == CB_CLAMP) *memo = v;
  }
  if (Q.flags & CB_MAPID) {
    const MapProbe2 pk = map_first_probe2(c.itab, Q.map_a, Q.map_m, v);
    bool mi;
    int64_t mv = map_sel2(pk, v, Q.map_def, &mi);
    if (__any_sync(0xffffffffu, mi)) mv = mi ? map_lookup_from2(c.itab, Q.map_a, Q.map_m, Q.map_def, v, pk) : mv;
    v = (valid || (Q.nullm & CB_MAPID)) ? mv : v;
    if (Q.memo == CB_MAPID) *memo = v;
  }
  if (Q.flags & CB_SIGRID) {
    const int64_t t = (int64_t)reduce_M(splitmix_H(Q.hs ^ (uint64_t)v), Q.M);
    v = (valid || (Q.nullm & CB_SIGRID)) ? t : v;
    if (Q.memo == CB_SIGRID) *memo = v;
  }
  if (Q.flags & CB_BUCKET) {
    int j0 = 0;
    const long long* m0 = l0 + Q.bk_row * 16;
    for (int k = 0; k < (Q.bk_m >> 6); ++k) j0 += v >= m0[k];
    const int64_t t = upper_bound_64(c.itab + Q.bk_a, Q.bk_m, smp[Q.bk_row], j0, v);
    v = (valid || (Q.nullm & CB_BUCKET)) ? t : v;
    if (Q.memo == CB_BUCKET) *memo = v;
  }
  stv_if(L > 0 && P0 < c.values_cap, c, P0, v);
}

// First id of a canonical output's row (0-id rows read a word of the plan blob).
template <class P>
__device__ __forceinline__ int64_t jl_prefetch(const P& p, const RbSmem& s, const JLCanon& Q, int r, bool in) {
  const RbRow Y = rb_row_p<kRbPitch>(s, Q.slot, r);
  const bool ok = in && Y.valid && Y.b > Y.a;
  return rap_ldin(ok ? p.val[Q.col] + Y.a : p.c.itab);
}

// An NGram output (R7) over K memoised provider words, n-windows: returns
// true when the row needs the generic path (late).
template <int K, int N, bool kSmall, class P>
__device__ __forceinline__ bool jl_ngram(const P& p, const RbSmem& s, const JLNgram<K>& G, const int64_t* mm,
                                         const int32_t* ml, int r, int wi, int lane, bool in, int64_t row, int64_t B,
                                         bool& ovf) {
  const Common& c = p.c;
  int32_t l[K];
  long long tot = 0;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    const RbRow X = rb_row_p<kRbPitch>(s, G.slot[i], r);
    l[i] = X.valid ? max(X.b - X.a, 0) : G.ncap[i];
    l[i] = min(l[i], G.cap[i]);
    tot += l[i];
  }
  const int32_t L = in ? (int32_t)min(max(tot - (long long)N + 1, 0ll), (long long)G.out_cap) : 0;
  const long long P0 = s.wb[G.q * 8 + wi] + rb_warp_excl<kSmall>(L, lane);
  stg_s32_if(in, c.lengths + ((int64_t)G.f * B + row), L);
  stg_s64_if(in, c.offsets + ((int64_t)G.f * B + row), P0);
  if (G.last) stg_s64_if(in && row == B - 1, c.offsets + (int64_t)(G.f + 1) * B, P0 + L);
  ovf |= P0 + L > c.values_cap;
  bool fast = true;
#pragma unroll
  for (int i = 0; i < K; ++i) fast = fast && l[i] <= 1 && (l[i] == 0 || ml[i] >= 1);
  uint64_t w[N];
#pragma unroll
  for (int j = 0; j < N; ++j) w[j] = 0;
  int32_t cnt = 0;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    const bool pr = l[i] != 0;
#pragma unroll
    for (int j = 0; j + 1 < N; ++j) w[j] = pr ? w[j + 1] : w[j];
    w[N - 1] = pr ? (uint64_t)mm[i] : w[N - 1];
    cnt += pr;
    if (i + 1 >= N) {
      uint64_t h = G.hsalt;
#pragma unroll
      for (int j = 0; j < N; ++j) h = splitmix_H(h ^ w[j]);
      const int64_t v = (int64_t)reduce_M(h, G.M);
      const long long at = P0 + (cnt - N);
      stv_if(fast && pr && cnt >= N && cnt - N < L && at < c.values_cap, c, at, v);
    }
  }
  return !fast && L > 0;
}

// Length and first position of an NGram row (the late path's recomputation).
template <int K, int N, bool kSmall>
__device__ __forceinline__ void jl_ngram_lp(const RbSmem& s, const JLNgram<K>& G, int r, int wi, int lane, bool in,
                                            int32_t* L, long long* P0) {
  long long tot = 0;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    const RbRow X = rb_row_p<kRbPitch>(s, G.slot[i], r);
    tot += min(X.valid ? max(X.b - X.a, 0) : G.ncap[i], G.cap[i]);
  }
  *L = in ? (int32_t)min(max(tot - (long long)N + 1, 0ll), (long long)G.out_cap) : 0;
  *P0 = s.wb[G.q * 8 + wi] + rb_warp_excl<kSmall>(*L, lane);
}

// Phase (3) by one warp (the generated kernel's first dense warp, while the
// sparse warps run pre_emit): wait until every CTA announced its totals,
// then each output's first offset for the block (as rows_body's phase 3) and
// the per-block capacity check.  blk totals: the CTA's s.ws sums.
template <bool kSmall>
__device__ __forceinline__ void rb_bases_warp(const Common& c, const RbGeom& g, const RbSmem& s, const int16_t* fidx,
                                              int FL, int fmax, int rb, int n_rb, int kws, long long chain0,
                                              const unsigned long long* pub, int lane) {
  if (lane == 0) {
    int ns = 32;
    while (ld_acquire(pub) < (unsigned long long)gridDim.x) {
      __nanosleep(ns);
      ns = min(ns * 2, 256);
    }
  }
  __syncwarp();
  long long* sT = reinterpret_cast<long long*>(s.dense);  // [fmax + 1]
  long long* sL = sT + (fmax + 1);                          // [fmax + 1]
  for (int f = lane; f <= fmax; f += 32) sT[f] = (long long)__ldcg(g.tot + f);
  const int nsb = rb / kRbSup, rb0 = nsb * kRbSup;
  constexpr int kBU = RAP_BASES_UNROLL;  // outputs whose lower-block loads are in flight together
  for (int f0 = 0; f0 <= fmax; f0 += kBU) {
    long long v[kBU];
#pragma unroll
    for (int u = 0; u < kBU; ++u) {
      const int f = min(f0 + u, fmax);
      long long a = 0;
      if (lane < nsb) a = (long long)__ldcg(g.sup + (int64_t)f * kRbSupMax + lane);
      if (rb0 + lane < rb) a += (long long)__ldcg(g.agg + (int64_t)f * n_rb + rb0 + lane);
      v[u] = a;
    }
#pragma unroll
    for (int u = 0; u < kBU; ++u) {
      const long long t = rb_warp_sum<kSmall>(v[u]);
      if (lane == 0 && f0 + u <= fmax) sL[f0 + u] = t;
    }
  }
  __syncwarp();
  long long P = chain0;
  for (int f0 = 0; f0 <= fmax; f0 += 32) {
    const int f = f0 + lane;
    const long long t = f <= fmax ? sT[f] : 0ll;
    long long x = t;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const long long y = __shfl_up_sync(0xffffffffu, x, d);
      if (lane >= d) x += y;
    }
    if (f <= fmax) sT[f] = P + x - t;
    P += __shfl_sync(0xffffffffu, x, 31);
  }
  __syncwarp();
  for (int fl = lane; fl < FL; fl += 32) {
    const int f = fidx[fl];
    long long blk = 0;
    for (int w = 0; w < kws; ++w) blk += s.ws[fl * 8 + w];
    s.base[fl] = sT[f] + sL[f];
    if (sT[f] + sL[f] + blk > c.values_cap) atomicExch(c.err, 1);  // values_capacity understated (sp_nnz)
  }
  __syncwarp();
}

// Context of one CTA: its feature group (processing indices [pb, pe)) and
// row block [R0, R1).
struct RbCtx {
  int pb, pe, FL, grp, rb, F, n_cols;
  int64_t B, R0, R1;
  const int16_t* slot;  // raw sparse column -> staged slot
  const int16_t* fidx;  // [FL] output index of processing index pb + fl
};

// The row-block kernel, parameterised by how an output's lengths and ids are
// evaluated (Pol): the built-in interpreter (rap_rows_interp.cuh) or the code
// generated for the plan (rap_jit.cpp).  Pol provides
//   setup(p, s, x)                   per-CTA records (threads < FL)
//   lengths<kSmall>(p, s, x, nr, acc) -> s.ws warp sums of every output
//   emit<kSmall>(p, s, x, c0, nr)     lengths, offsets, ids of the chunk
template <class Pol, int MD, int MS, bool kSmall>
__device__ __forceinline__ void rows_body(const RbParams<MD, MS>& p) {
  unsigned char* const smem = rap_dyn_smem;
  __shared__ CtaState cs;
  __shared__ int16_t s_slot[MS];  // raw sparse column -> staged slot (-1: not staged)
  __shared__ int16_t s_cols[MS];  // staged slot -> raw sparse column
  __shared__ unsigned long long s_mask[(MS + 63) / 64];
  __shared__ int16_t s_fidx[kJitMaxF > kRbMaxFL ? kJitMaxF : kRbMaxFL];
  __shared__ int s_last, s_fmax;
  __shared__ uint64_t s_sbar;  // staging mbarrier (bulk copies)
  __shared__ int s_sphase;
  __shared__ uint64_t s_ibar;  // id staging mbarrier (generated kernel, g.id_slots > 0)
  __shared__ int s_iphase;
  const RbGeom& g = p.g;
  const Common& c = p.c;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // generated kernel with a dense warp: warps 0-6 run the sparse phases over
  // 224-row chunks while warp 7 evaluates the dense outputs of the block
  constexpr bool kDW = Pol::kDenseWarp;
  // generated kernel in warp-pair mode (Pol::kPairs, 512-thread CTAs): warps
  // 2w and 2w + 1 evaluate two halves of the outputs over the same 32 rows of
  // a 224-row chunk, so each row has two threads (twice the warps per SM at
  // <= 64 registers, the row blocks as in the one-thread-per-row form)
  constexpr int kT = Pol::kThreads;                                 // threads per CTA
  constexpr int kTS = Pol::kPairs ? 224 : (kDW ? 224 : kRbChunk);  // rows per chunk
  constexpr int kWS = kTS / 32;                                    // row warps (s.ws / s.wb columns)
  constexpr int kNW = kDW ? 7 : kT / 32;                           // warps running the sparse phases
  RbCtx x;
  x.F = c.n_sparse_out;
  const RbSmem s = rb_carve(smem, g, x.F);
  const int n_rb = g.n_rb;
  // CTAs [n_rb * n_fg, + n_dcta) evaluate only dense blocks (small batches:
  // the dense work runs beside the sparse phases instead of after them)
  const int n_sc = n_rb * g.n_fg;
  const bool dcta = (int)blockIdx.x >= n_sc;
  x.grp = dcta ? 0 : (int)blockIdx.x / n_rb;
  x.rb = dcta ? 0 : (int)blockIdx.x - x.grp * n_rb;
  x.pb = dcta ? 0 : g.fg_off[x.grp];
  x.pe = dcta ? 0 : g.fg_off[x.grp + 1];
  x.FL = x.pe - x.pb;
  x.B = c.n_rows;
  x.R0 = (int64_t)x.rb * g.rows_rb;
  x.R1 = dcta ? x.R0 : min(x.B, x.R0 + (int64_t)g.rows_rb);
  x.slot = s_slot;
  x.fidx = s_fidx;
  const int FL = x.FL, rb = x.rb;
  const int nrows = (int)max((int64_t)0, x.R1 - x.R0);
  const int nch = (nrows + kTS - 1) / kTS;
  unsigned long long* const pub = g.sched + 2;  // CTAs whose totals are stored
  // programmatic dependent launch (Pol::kPDL): the next launch on the stream
  // may start its CTAs as this one's leave the SMs; before reading any data
  // a previous launch may have written (its inputs, the chained offsets, the
  // counters) it waits for the previous grid (griddepcontrol.wait below), so
  // only the CTA setup overlaps the previous launch's tail
  if (Pol::kPDL) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  trace_stamp(c, 0);

  if (tid == 0) {
    mbar_init(&cs.bar, 1);
    s_sphase = 0;
    s_iphase = 0;
    cs.phase = 0;
    cs.dgroup = -1;
    s_fmax = 0;
    if (blockIdx.x == 0 && x.F == 0 && !c.chain && c.offsets) c.offsets[0] = 0;  // no sparse outputs (R17)
  }
  for (int i = tid; i < (MS + 63) / 64; i += kT) s_mask[i] = 0ull;
  __syncthreads();
  // the raw columns the group reads -> staged slots (one group of every
  // output: the plan's column mask, no per-output loads)
  const bool all = x.pb == 0 && x.pe == x.F;
  if (tid < FL) {
    const int f = __ldg(g.perm + x.pb + tid);
    s_fidx[tid] = (int16_t)f;
    if (!all) {
      atomicMax(&s_fmax, f);
      const RbFeat& G = g.feat[f];
      const int kk = __ldg(&G.kind) == 1 ? 0 : __ldg(&G.k);
      for (int i = 0; i < kk; ++i) {
        const int src = __ldg(&G.src[i]);
        if (src >= 0) atomicOr(&s_mask[src >> 6], 1ull << (src & 63));
      }
    }
  }
  if (all && tid == 0) {
    s_fmax = x.F - 1;
    s_mask[0] = g.all_cols;
  }
  __syncthreads();
  int n_cols = 0;
  for (int i = 0; i < (MS + 63) / 64; ++i) n_cols += __popcll(s_mask[i]);
  x.n_cols = n_cols;
  if (tid == 0) mbar_init(&s_sbar, (uint32_t)max(n_cols, 1));  // staging: one arrival per column
  // id staging: one arrival per slot < n_ids, issued with the chunk's offsets
  // (phase 1 when the block is one chunk, else phase 4) and awaited just
  // before the chunk's ids are emitted
  const int n_ids = min(n_cols, g.id_slots);
  if (tid == 0) mbar_init(&s_ibar, (uint32_t)max(n_ids, 1));
  for (int col = tid; col < MS; col += kT) {
    const unsigned long long m = s_mask[col >> 6];
    int before = __popcll(m & ((1ull << (col & 63)) - 1ull));
    for (int i = 0; i < (col >> 6); ++i) before += __popcll(s_mask[i]);
    const bool on = (m >> (col & 63)) & 1ull;
    s_slot[col] = on ? (int16_t)before : (int16_t)-1;
    if (on) s_cols[before] = (int16_t)col;
  }
  __syncthreads();
  if (Pol::kPDL) asm volatile("griddepcontrol.wait;" ::: "memory");  // the previous launch's grid is done
  const long long chain0 = c.chain ? (long long)__ldcg(c.offsets) : 0ll;
  trace_stamp(c, 6);
  if (Pol::kSetupEarly) {
    Pol::setup(p, s, x);
    __syncthreads();
  }
  trace_stamp(c, 7);
  if (kDW && warp >= kWS) {
    // Pol::kDenseLate: the dense warps start once the sparse warps announced
    // the block's totals (named barrier 2), so the staging and length phases
    // on the critical path do not share the SM's issue slots with them
    if (Pol::kDenseLate) asm volatile("bar.sync 2, %0;" ::"r"(kT) : "memory");
    if (Pol::kBasesByDense && warp == kWS && FL > 0 && nrows > 0) {
      // phase (3) for the sparse warps, while they run pre_emit: their
      // per-output sums (s.ws) are visible after named barrier 4, the bases
      // are handed back on named barrier 3
      asm volatile("bar.sync 4, %0;" ::"r"(kTS + 32) : "memory");
      rb_bases_warp<kSmall>(c, g, s, s_fidx, FL, s_fmax, rb, n_rb, kWS, chain0, pub, lane);
      trace_stamp_warp(c, 4);
      asm volatile("bar.arrive 3, %0;" ::"r"(kTS + 32) : "memory");
    }
    Pol::dense_warp(p, s, x);  // the dense outputs of rows [R0, R1), concurrent with the sparse phases
    trace_stamp_warp(c, 15);
    if (Pol::kTail && nch == 1 && FL > 0 && nrows > 0) {
      // the tail outputs of every row warp, once the sparse warps set the
      // chunk's warp bases (named barrier 5)
      constexpr int kND = kT / 32 - kWS;  // dense warps
      asm volatile("bar.sync 5, %0;" ::"r"(kT) : "memory");
      for (int w = warp - kWS; w < kWS; w += kND) Pol::template emit_tail<kSmall>(p, s, x, x.R0, nrows, w);
    }
  } else {

  // (1) per-output totals of my rows -> agg, then announce the CTA
  for (int ch = 0; ch < nch; ++ch) {
    const int64_t c0 = x.R0 + (int64_t)ch * kTS;
    const int nr = (int)min((int64_t)kTS, x.R1 - c0);
    rb_stage<kDW>(p, s, s_cols, n_cols, c0, nr, &s_sbar, &s_sphase, nch == 1 ? n_ids : 0, &s_ibar);
    if (ch == 0) trace_stamp(c, 8);
    Pol::template lengths<kSmall>(p, s, x, nr, ch > 0);
    rb_sync<kDW>();
  }
  long long blk_tot = 0;  // thread tid < FL: output tid's ids in this block
  if (tid < FL) {
    long long tot = 0;
    if (nch > 0)
#pragma unroll
      for (int w = 0; w < kWS; ++w) tot += s.ws[tid * 8 + w];
    blk_tot = tot;
    const int f = s_fidx[tid];
    g.agg[(int64_t)f * n_rb + rb] = (unsigned long long)tot;  // feature-major: row blocks of f contiguous
    atomicAdd(g.tot + f, (unsigned long long)tot);           // red.add: the output's total over all blocks
    atomicAdd(g.sup + (int64_t)f * kRbSupMax + rb / kRbSup, (unsigned long long)tot);  // and its super block's
  }
  trace_stamp(c, 13);
  rb_sync<kDW>();
  if (tid == 0) {
    __threadfence();  // release: the block's totals before the announcement
    atomicAdd(pub, 1ull);
  }
  if (kDW && Pol::kDenseLate) asm volatile("bar.arrive 2, %0;" ::"r"(kT) : "memory");  // the dense warps may start
  constexpr bool kDB = kDW && Pol::kBasesByDense;  // phase (3) by the first dense warp
  if (kDB && FL > 0 && nrows > 0) asm volatile("bar.arrive 4, %0;" ::"r"(kTS + 32) : "memory");
  trace_stamp(c, 1);

  if (!Pol::kSetupEarly) Pol::setup(p, s, x);  // records used only in (4)

  // a one-chunk block: the policy's first outputs' values (everything but
  // their positions) computed now, so the wait below and the base loads
  // overlap them (the generated policy's pre_emit; carried in registers)
  typename Pol::PreState pre{};
  const bool use_pre = Pol::kPre && nch == 1 && FL > 0 && nrows > 0;
  if (use_pre) pre = Pol::pre_emit(p, s, x, x.R0, nrows);

  // (2) dense outputs (independent of the scan): the policy's own rows-of-this-
  // block code when it has one and the dense rows are the batch rows, else the
  // launch's dense blocks round robin over the CTAs (the dense warp took them)
  if (!kDW) {
    if (Pol::kGenDense && all && c.dense_row0 == 0 && c.n_dense_rows == c.n_rows && c.n_groups > 0) {
      Pol::dense(p, s, x);
    } else {
      const int64_t d0 = g.n_dcta ? (int64_t)blockIdx.x - n_sc : (int64_t)blockIdx.x;
      const int64_t dstep = g.n_dcta ? (int64_t)g.n_dcta : (int64_t)gridDim.x;
      for (int64_t d = d0; d >= 0 && d < c.n_dense_tiles; d += dstep) {
        const uint32_t gi = (uint32_t)d % (uint32_t)c.n_groups;
        dense_block(p, (int)gi, (int64_t)((uint32_t)d / (uint32_t)c.n_groups), 0, cs);
        __syncthreads();
        if (d == d0) trace_stamp(c, 9);
      }
    }
  }
  rb_sync<kDW>();
  trace_stamp(c, 2);

  if (FL > 0 && nrows > 0) {
    if (kDB) {
      asm volatile("bar.sync 3, %0;" ::"r"(kTS + 32) : "memory");  // the dense warp's bases
    } else {
    // (3) wait until every CTA announced its totals (all resident: cooperative launch)
    if (tid == 0) {
      int ns = 32;
      while (ld_acquire(pub) < (unsigned long long)gridDim.x) {
        __nanosleep(ns);
        ns = min(ns * 2, 256);
      }
    }
    rb_sync<kDW>();
    trace_stamp(c, 3);
    // T[f] = the output's total (red.add into g.tot), L[f] = its ids in the
    // row blocks below mine: the super blocks below mine (32 row blocks each,
    // red.add totals) plus the row blocks of my super block below mine -- one
    // coalesced load per lane for each, whatever n_rb (warp w reduces
    // outputs w, w + kWS, ..., four at a time so their loads are in flight together)
    const int fmax = s_fmax;
    long long* sT = reinterpret_cast<long long*>(s.dense);  // [fmax + 1]
    long long* sL = sT + (fmax + 1);                          // [fmax + 1]
    for (int f = tid; f <= fmax; f += kNW * 32) sT[f] = (long long)__ldcg(g.tot + f);
    {
      const int nsb = rb / kRbSup, rb0 = nsb * kRbSup;
      for (int f0 = warp; f0 <= fmax; f0 += 4 * kNW) {
        long long v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int f = min(f0 + u * kNW, fmax);
          long long a = 0;
          if (lane < nsb) a = (long long)__ldcg(g.sup + (int64_t)f * kRbSupMax + lane);
          if (rb0 + lane < rb) a += (long long)__ldcg(g.agg + (int64_t)f * n_rb + rb0 + lane);
          v[u] = a;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const long long t = rb_warp_sum<kSmall>(v[u]);
          if (lane == 0 && f0 + u * kNW <= fmax) sL[f0 + u * kNW] = t;
        }
      }
    }
    trace_stamp(c, 10);
    rb_sync<kDW>();
    trace_stamp(c, 11);
    trace_stamp(c, 12);
    if (warp == 0) {  // exclusive prefix over outputs in feature-major order (warp scan, 32 at a time)
      long long P = chain0;
      for (int f0 = 0; f0 <= fmax; f0 += 32) {
        const int f = f0 + lane;
        const long long t = f <= fmax ? sT[f] : 0ll;
        long long x = t;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const long long y = __shfl_up_sync(0xffffffffu, x, d);
          if (lane >= d) x += y;
        }
        if (f <= fmax) sT[f] = P + x - t;
        P += __shfl_sync(0xffffffffu, x, 31);
      }
    }
    rb_sync<kDW>();
    if (tid < FL) {
      const int f = s_fidx[tid];
      s.base[tid] = sT[f] + sL[f];
      // values_capacity (from sp_nnz) understated: an output's ids of this
      // block end past it (the emitters store nothing past it; one check per
      // output and block instead of one per row)
      if (sT[f] + sL[f] + blk_tot > c.values_cap) atomicExch(c.err, 1);
    }
    rb_sync<kDW>();
    trace_stamp(c, 4);
    }  // phase (3) by the sparse warps

    // (4) lengths, offsets and ids, chunk by chunk
    for (int ch = 0; ch < nch; ++ch) {
      const int64_t c0 = x.R0 + (int64_t)ch * kTS;
      const int nr = (int)min((int64_t)kTS, x.R1 - c0);
      if (nch > 1) {
        rb_stage<kDW>(p, s, s_cols, n_cols, c0, nr, &s_sbar, &s_sphase, n_ids, &s_ibar);
        Pol::template lengths<kSmall>(p, s, x, nr, false);
        rb_sync<kDW>();
      }
      if (tid < FL) {  // warp bases of this chunk; the running base advances
        long long b = s.base[tid];
#pragma unroll
        for (int w = 0; w < kWS; ++w) {
          s.wb[tid * 8 + w] = b;
          b += s.ws[tid * 8 + w];
        }
        s.base[tid] = b;
      }
      rb_sync<kDW>();
      if (n_ids > 0) mbar_wait(&s_ibar, (uint32_t)s_iphase);  // the chunk's staged ids landed
      const bool tail = kDW && Pol::kTail && nch == 1;  // the dense warps emit the tail outputs
      if (tail) asm volatile("bar.arrive 5, %0;" ::"r"(kT) : "memory");  // (warp bases set above)
      Pol::template emit<kSmall>(p, s, x, c0, nr, pre, use_pre && ch == 0, tail);
      rb_sync<kDW>();
      if (n_ids > 0 && tid == 0) s_iphase ^= 1;
    }
  }
  }  // sparse warps
  trace_stamp(c, 5);

  // last CTA out: reset the counters (launch parameters stay the same)
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    const unsigned long long prev = atomicAdd(g.sched, 1ull);
    s_last = (prev == (unsigned long long)gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  if (s_last) {
    __threadfence();
    for (int f = tid; f < x.F; f += kT) g.tot[f] = 0ull;
    const int nsb_all = (n_rb + kRbSup - 1) / kRbSup;
    for (int i = tid; i < x.F * nsb_all; i += kT) g.sup[(int64_t)(i / nsb_all) * kRbSupMax + i % nsb_all] = 0ull;
    if (tid == 0) {
      g.sched[0] = 0ull;
      g.sched[2] = 0ull;
    }
    __threadfence();
  }
  trace_stamp(c, 14);
}

}  // namespace rapk
