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

#include <map>
#include <mutex>
#include <utility>

#include "rap_internal.h"
#include "rap_device.cuh"

namespace rapk {

__host__ __device__ constexpr int align_up_c(int x, int a) { return (x + a - 1) / a * a; }

template <int MD, int MS>
struct KParams {
  Common c;
  const float* dense[MD];
  const uint32_t* dvalid[MD];
  const int32_t* off[MS];
  const int64_t* val[MS];
  const uint32_t* svalid[MS];
};

#ifndef RAP_LBATCH
#define RAP_LBATCH 8
#endif
constexpr int kLBatch = RAP_LBATCH;  // tiles per batch of the length pass
constexpr int kGroups = kTileRows / 32;  // row groups of a sparse tile (one row per lane each)
// Warp-private shared memory of the sparse phases: the NGram
// paths use its first 4 KB; the canonical paths stage Arrow offsets,
// validity words and ids in it with cp.async (nothing in flight in registers).
#ifndef RAP_WARP_SCR
#define RAP_WARP_SCR 6656
#endif
constexpr int kWarpScr = RAP_WARP_SCR;  // 8 warps x 6.5 KB: 4 CTAs fit an SM's 228 KB
constexpr int kNgScratch = kWarps * kWarpScr;
static_assert(4 * kMaxNgramK * 32 * 4 <= kWarpScr, "NGram scratch exceeds the warp region");
constexpr int kLChunkTiles = 8;  // length pass: tiles staged per round
constexpr int kVChunkTiles = 4;  // value pass: tiles staged per round
#ifndef RAP_VGROUP
#define RAP_VGROUP 1
#endif
constexpr int kVGroup = RAP_VGROUP;  // value pass: tiles whose elements run the pipeline together
constexpr int kLStageOff = 0, kLStageBm = align_up_c((kLChunkTiles * 128 + 4) * 4, 16);
constexpr int kVStageOff = 0, kVStageBm = align_up_c((kVChunkTiles * 128 + 4) * 4, 16);
constexpr int kVStageId = kVStageBm + kVChunkTiles * 128 / 32 * 4;
static_assert(kLStageBm + kLChunkTiles * 4 * 4 <= kWarpScr, "length-pass staging exceeds the warp region");
static_assert(kVStageId + kVChunkTiles * 128 * 8 <= kWarpScr && kVStageId % 16 == 0, "value-pass staging layout");
// Aggregate word of a CTA: [63:44] tag = launch epoch + 1 (0 = never
// written), [43:0] the CTA's output length total.
constexpr int kEpochShift = 44;
constexpr unsigned long long kValueMask = (1ull << kEpochShift) - 1;
constexpr unsigned long long kEpochMax = (1ull << 20) - 2;


// ----------------------------------------------------------------------------
// Jagged scan (R17) over the feature-major sparse tile sequence.  Each CTA
// owns a contiguous, cost-balanced range of it (host partition, DESIGN.md
// §7) and splits it into one contiguous sub-range per warp.  Phase L sums
// every sub-range's output lengths (closed form from the Arrow offsets) and
// publishes the CTA aggregate; after its dense blocks the CTA adds its
// predecessors' aggregates (one parallel read, no chained look-back), so
// every warp knows the base of its sub-range before it stores anything and
// then walks its tiles with a running base: a tile function takes its base
// and returns its output length total.
// Per-feature dispatch state a warp keeps in registers across its tiles.
enum TileKind : int { TK_CANON = 0, TK_NGRAM_FAST = 1, TK_NGRAM = 2, TK_GENERIC = 3 };
struct FeatCtx {
  int f, kind, sk, src, has_fill, ng_staged;
  int64_t xcap, null_xcap, fill;
  Canon q;  // canonical pipeline (TK_CANON), in registers
};

__device__ __forceinline__ int64_t clamp_tile(int64_t t, int64_t lo, int64_t hi) { return t < lo ? lo : (t > hi ? hi : t); }

template <class P>
__device__ __forceinline__ void load_ctx(const P& p, int f, FeatCtx& x) {
  const SProg& pg = p.c.sprogs[f];
  const Chain ch = pg.ch;  // one burst of independent loads
  x.q = pg.cn;
  x.f = f;
  x.sk = ch.src_kind;
  x.src = ch.src;
  x.has_fill = ch.has_fill;
  x.xcap = ch.xcap;
  x.null_xcap = ch.null_xcap;
  x.fill = ch.fill;
  x.ng_staged = 0;
  if (x.sk == SRC_SPARSE) {
    x.kind = x.q.ok ? TK_CANON : TK_GENERIC;
  } else if (x.sk == SRC_NGRAM) {
    const int k = pg.ng.k;
    bool fast = x.q.ok && k <= 4;
    for (int c = 0; c < k; ++c) fast = fast && pg.src_cn[c].ok && pg.src[c].src_kind == SRC_SPARSE;
    x.kind = fast ? TK_NGRAM_FAST : TK_NGRAM;
  } else {
    x.kind = TK_GENERIC;
  }
  __syncwarp();
}

// Arrow offsets of rows r0+4*lane .. +4 and the validity word of those rows.
struct Quad {
  int32_t a[5];
  uint32_t w;
};

// Called by the whole warp (the fifth offset of lane i is lane i+1's first,
// by shuffle: one 16-byte load per lane plus one scalar load for lane 31).
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
  } else {
#pragma unroll
    for (int k = 0; k < 4; ++k) q.a[k] = row + k <= B ? __ldg(off + row + k) : 0;
  }
  const int32_t last = (lane == 31 && row + 4 <= B) ? __ldg(off + row + 4) : 0;
  q.w = (bm != nullptr && row < B) ? __ldg(bm + (row >> 5)) : 0xffffffffu;
  const int32_t nxt = __shfl_down_sync(0xffffffffu, q.a[0], 1);
  q.a[4] = lane == 31 ? last : nxt;
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

// Stage the Arrow offsets off[R0 .. R0+NR] and the validity words of rows
// [R0, R0+NR) (R0 a multiple of 32) into warp shared memory with cp.async;
// the caller waits (cp_async_wait_all) and __syncwarp()s before reading.
__device__ __forceinline__ void stage_offsets(const int32_t* off, const uint32_t* bm, int64_t R0, int NR, int32_t* soff,
                                              uint32_t* sbm, int lane) {
  const int ne = NR + 1;
  int done = 0;
  if ((reinterpret_cast<uintptr_t>(off + R0) & 15) == 0) {
    const int n16 = ne >> 2;
    for (int i = lane; i < n16; i += 32) cp_async16(soff + 4 * i, off + R0 + 4 * i);
    done = n16 * 4;
  }
  for (int i = done + lane; i < ne; i += 32) cp_async4(soff + i, off + R0 + i);
  const int nw = (NR + 31) >> 5;
  if (bm != nullptr) {
    for (int i = lane; i < nw; i += 32) cp_async4(sbm + i, bm + (R0 >> 5) + i);
  } else {
    for (int i = lane; i < nw; i += 32) sbm[i] = 0xffffffffu;
  }
}

// Output length of staged local row lr (R5 FirstX cap, R10 fill, R14 null).
__device__ __forceinline__ int32_t len_s(const int32_t* soff, const uint32_t* sbm, int lr, int64_t xcap, int has_fill,
                                         int64_t null_xcap) {
  if ((sbm[lr >> 5] >> (lr & 31)) & 1u) return (int32_t)min((int64_t)max(soff[lr + 1] - soff[lr], 0), xcap);
  return has_fill ? (int32_t)min((int64_t)1, null_xcap) : 0;
}

// ----------------------------------------------------------------------------
// Phase 3: offsets and ids of sparse tile (f, rt), whose first output id goes
// to values[base].
template <class P>
__device__ __noinline__ void value_group_general(const P& p, int f, int64_t row0, int lane, int32_t mylen,
                                                 int32_t myst, int32_t lx, long long gbase);
template <class P>
__device__ __noinline__ long long value_tile_ngram(const P& p, int f, int64_t rt, int lane, long long base,
                                                   int32_t* scr);

// Output stores are streaming (st.global.cs, evict-first in L2): written once,
// never read back by the kernel.
__device__ __forceinline__ void st_cs64(int64_t* p, int64_t v) { __stcs(reinterpret_cast<long long*>(p), (long long)v); }
// A value of the jagged output (R17) in the launch's value type: int64, or
// int32 under Cast (RAP_OUT_VALUES_I32, two's-complement truncation).
__device__ __forceinline__ void st_val(int64_t* values, bool i32, long long pos, int64_t v) {
  if (i32)
    __stcs(reinterpret_cast<int*>(values) + pos, (int)v);
  else
    st_cs64(values + pos, v);
}

// Lengths (int4) and offsets (2 x longlong2) of the lane's 4 rows.
__device__ __forceinline__ void store_quad(int32_t* lp, int64_t* op, int64_t row, int64_t B, const int32_t* l,
                                           long long lb, const int32_t* e) {
  if (row + 4 <= B && (reinterpret_cast<uintptr_t>(lp) & 15) == 0 && (reinterpret_cast<uintptr_t>(op) & 15) == 0) {
    __stcs(reinterpret_cast<int4*>(lp), make_int4(l[0], l[1], l[2], l[3]));
    __stcs(reinterpret_cast<longlong2*>(op), make_longlong2(lb + e[0], lb + e[1]));
    __stcs(reinterpret_cast<longlong2*>(op) + 1, make_longlong2(lb + e[2], lb + e[3]));
  } else {
#pragma unroll
    for (int k = 0; k < 4; ++k)
      if (row + k < B) {
        __stcs(lp + k, l[k]);
        st_cs64(op + k, lb + e[k]);
      }
  }
}

// Tile of a canonical SRC_SPARSE chain; the lane owns rows r0 + 4*lane + k,
// so its output ids are contiguous.
template <class P>
__device__ __noinline__ long long value_tile_canon(const P& p, const FeatCtx& fc, int64_t rt, int lane,
                                                      long long base) {
  const Canon& q = fc.q;
  const int f = fc.f;
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rt * kTileRows;
  const int64_t row = r0 + 4 * lane;
  int64_t* values = p.c.values;
  const bool vi32 = p.c.vi32 != 0;  // Cast: int32 values (RAP_OUT_VALUES_I32)
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
  const bool last = f == p.c.n_sparse_out - 1 && rt == p.c.tiles_per_feature - 1;
  int32_t* lp = p.c.lengths + (int64_t)f * B + row;
  int64_t* op = p.c.offsets + (int64_t)f * B + row;
  if (__all_sync(0xffffffffu, l[0] <= 1 && l[1] <= 1 && l[2] <= 1 && l[3] <= 1)) {
    // at most one id per row: the ids are computed before the base is known
    int64_t v[4];
    unsigned act = 0, full = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      act |= (l[k] == 1 ? 1u : 0u) << k;
      full |= (quad_valid(qd, k, lane) ? 1u : 0u) << k;
      v[k] = (l[k] == 1 && quad_valid(qd, k, lane)) ? __ldg(val + qd.a[k]) : fc.fill;
    }
    canon_apply_n<4>(q, itab, v, act, full);
    const long long lb = base + L;
    store_quad(lp, op, row, B, l, lb, e);
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const long long pos = lb + e[k];
      if (l[k] == 1 && pos < cap) st_val(values, vi32, pos, v[k]);
    }
    if (last && lane == 31) {
      p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + T;  // total, R17
      if (base + T > cap) atomicExch(p.c.err, 1);
    }
    return T;
  }
  store_quad(lp, op, row, B, l, base + L, e);
  if (last && lane == 31) {
    p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + T;
    if (base + T > cap) atomicExch(p.c.err, 1);
  }
  // multi-id rows: elements in output order, 128 per round (4 per lane, all
  // loads in flight together); owning lane by a 5-step shuffle search over
  // the lane prefixes, then the row within the lane
  const int mylex = L;
  for (int eb = 0; eb < T; eb += 128) {
    int64_t x[4];
    unsigned act = 0, full = 0;
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int ee = eb + 32 * u + lane;
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
      const bool au = ee < T, fu = (wr >> ((4 * r + k) & 31)) & 1u;
      act |= (au ? 1u : 0u) << u;
      full |= (fu ? 1u : 0u) << u;
      x[u] = (au && fu) ? __ldg(val + ak + (in_lane - ek)) : fc.fill;
    }
    canon_apply_n<4>(q, itab, x, act, full);
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const long long pos = base + eb + 32 * u + lane;
      if (((act >> u) & 1u) && pos < cap) st_val(values, vi32, pos, x[u]);
    }
  }
  return T;
}

// Up to kVChunkTiles consecutive tiles rt0 .. rt0+nt-1 of a canonical chain:
// the offsets / validity words, then the ids of the chunk are staged in warp
// shared memory with cp.async (no loads in flight in registers), then the
// canonical pipeline runs 8 elements per lane at a time (MapId probes and
// Bucketize steps of 8 rows in flight together).  Eligible when every row
// has at most one output id; returns the chunk's output length total, or -1
// with nothing written otherwise.
template <class P>
__device__ __noinline__ long long value_chunk_canon(const P& p, const FeatCtx& fc, int64_t rt0, int nt, int lane,
                                                    long long base, unsigned char* wscr) {
  int32_t* soff = reinterpret_cast<int32_t*>(wscr + kVStageOff);
  uint32_t* sbm = reinterpret_cast<uint32_t*>(wscr + kVStageBm);
  int64_t* sid = reinterpret_cast<int64_t*>(wscr + kVStageId);
  const int f = fc.f;
  const int64_t B = p.c.n_rows;
  const int64_t R0 = rt0 * kTileRows;
  const int NR = (int)min((int64_t)nt * kTileRows, B - R0);
  const int src = fc.src;
  const int64_t xcap = fc.xcap, null_xcap = fc.null_xcap;
  const int has_fill = fc.has_fill;
  trace_clk(p.c, 8, 0);
  stage_offsets(p.off[src], p.svalid[src], R0, NR, soff, sbm, lane);
  cp_async_wait_all();
  __syncwarp();
  trace_clk(p.c, 9, soff[0]);
  // quad layout: the lane owns local rows j*128 + 4*lane + k; one 16-byte
  // and one 4-byte shared load give its 5 offsets, one word its 4 validity bits
  unsigned act = 0, full = 0;
  bool ok = true;
  const int xc = (int)min(xcap, (int64_t)INT32_MAX);
  const int nl = has_fill ? (int)min((int64_t)1, null_xcap) : 0;  // R10 / R14
#pragma unroll
  for (int j = 0; j < kVChunkTiles; ++j) {
    const int lr0 = j * kTileRows + 4 * lane;
    if (lr0 < NR) {
      const int4 a = *reinterpret_cast<const int4*>(soff + lr0);
      const int a4 = soff[lr0 + 4];
      const unsigned vb = (sbm[lr0 >> 5] >> (lr0 & 31)) & 15u;
      const int d[4] = {a.y - a.x, a.z - a.y, a.w - a.z, a4 - a.w};
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const bool in = lr0 + k < NR;
        const bool va = in && ((vb >> k) & 1u);
        const int l = !in ? 0 : (va ? min(max(d[k], 0), xc) : nl);  // R5 FirstX cap
        ok &= l <= 1;
        act |= (l == 1 ? 1u : 0u) << (4 * j + k);
        full |= (va ? 1u : 0u) << (4 * j + k);
      }
    }
  }
  if (!__all_sync(0xffffffffu, ok)) {
    __syncwarp();
    return -1;
  }
  const int64_t* val = p.val[src];
  const unsigned fetch = act & full;
#pragma unroll
  for (int j = 0; j < kVChunkTiles; ++j)
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int lr = j * kTileRows + 4 * lane + k;
      if ((fetch >> (4 * j + k)) & 1u) cp_async8(sid + lr, val + soff[lr]);
    }
  cp_async_wait_all();  // each lane reads only the ids it staged
  trace_clk(p.c, 10, sid[4 * lane]);
  int64_t* values = p.c.values;
  const bool vi32 = p.c.vi32 != 0;  // Cast: int32 values (RAP_OUT_VALUES_I32)
  const long long cap = p.c.values_cap;
  long long run = base;
  const int64_t* const itab_h = p.c.itab;  // hoisted (value_tile_multi)
#pragma unroll 1
  for (int j0 = 0; j0 < nt; j0 += kVGroup) {
    int64_t v[4 * kVGroup];
    const unsigned gm = (1u << (4 * kVGroup)) - 1u;
    const unsigned ag = (act >> (4 * j0)) & gm, fg = (full >> (4 * j0)) & gm;
#pragma unroll
    for (int u = 0; u < 4 * kVGroup; ++u) {
      const int lr = (j0 + (u >> 2)) * kTileRows + 4 * lane + (u & 3);
      v[u] = ((ag & fg) >> u) & 1u ? sid[lr] : fc.fill;
    }
    canon_apply_n<4 * kVGroup>(fc.q, itab_h, v, ag, fg);
    trace_clk(p.c, 11, v[0]);
#pragma unroll
    for (int jj = 0; jj < kVGroup; ++jj) {
      const int j = j0 + jj;
      if (j < nt) {
        const int64_t rt = rt0 + j;
        const int64_t row = rt * kTileRows + 4 * lane;
        const unsigned a4 = (ag >> (4 * jj)) & 15u;
        int32_t l[4], e[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          l[k] = (a4 >> k) & 1u;
          e[k] = __popc(a4 & ((1u << k) - 1u));
        }
        const int tot = __popc(a4);
        const int incl = warp_incl_scan(tot, lane);
        const int Tj = __shfl_sync(0xffffffffu, incl, 31);
        const long long lb = run + (incl - tot);
        store_quad(p.c.lengths + (int64_t)f * B + row, p.c.offsets + (int64_t)f * B + row, row, B, l, lb, e);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const long long pos = lb + e[k];
          if (l[k] && pos < cap) st_val(values, vi32, pos, v[4 * jj + k]);
        }
        if (f == p.c.n_sparse_out - 1 && rt == p.c.tiles_per_feature - 1 && lane == 31) {
          p.c.offsets[(int64_t)p.c.n_sparse_out * B] = run + Tj;  // total, R17
          if (run + Tj > cap) atomicExch(p.c.err, 1);
        }
        run += Tj;
      }
    }
  }
  trace_clk(p.c, 12, run);
  __syncwarp();  // the region is reused by the next chunk
  return run - base;
}

constexpr int kNullRow = INT_MIN;
#ifndef RAP_MULTI_DEPTH
#define RAP_MULTI_DEPTH 3
#endif
constexpr int kMultiDepth = RAP_MULTI_DEPTH;  // id windows in flight (ring of 4)
static_assert(kMultiDepth >= 1 && kMultiDepth <= 3, "ring of 4 window slots");
constexpr int kMultiRing = 1584;  // byte offset of the id ring in the warp scratch
static_assert(kMultiRing + 4 * 128 * 8 <= kWarpScr, "multi-id tile scratch");
// Tile rt of a canonical chain whose rows may hold several ids (multi-hot,
// FirstX caps): element-parallel.  Offsets / validity staged with cp.async.
// Output element e of a valid row r reads input e + delta_r, delta_r =
// soff[r] - out_start[r] (FirstX keeps a prefix, R5); a filled null row
// (R10) emits the fill id.  delta is constant over runs of consecutive valid
// rows that FirstX does not truncate, so the tile keeps only its *change
// points* (output position where delta changes, or a filled null's element)
// in shared memory: ~10 per 128 multi-hot rows instead of one per row.  Each
// 128-element window of the output (e = window + 32u + lane: coalesced id
// loads and value stores) takes the delta of the last change point at or
// before its start, then applies the few change points inside the window;
// ids are cp.async-staged into a 4-slot ring with kMultiDepth windows in
// flight.
template <bool I32, class P>  // I32: int32 values (Cast), a compile-time branch of the window loop
__device__ __noinline__ long long value_tile_multi(const P& p, const FeatCtx& fc, int64_t rt, int lane, long long base,
                                                   unsigned char* wscr) {
  int32_t* soff = reinterpret_cast<int32_t*>(wscr);        // [132]
  uint32_t* sbm = reinterpret_cast<uint32_t*>(wscr + 528);  // [4]
  int2* cps = reinterpret_cast<int2*>(wscr + 544);          // [128] change points (position, delta)
  const int f = fc.f;
  const int64_t B = p.c.n_rows;
  const int64_t R0 = rt * kTileRows;
  const int NR = (int)min((int64_t)kTileRows, B - R0);
  const int src = fc.src;
  stage_offsets(p.off[src], p.svalid[src], R0, NR, soff, sbm, lane);
  cp_async_wait_all();
  __syncwarp();
  const int xc = (int)min(fc.xcap, (int64_t)INT32_MAX);
  const int nl = fc.has_fill ? (int)min((int64_t)1, fc.null_xcap) : 0;  // R10 / R14
  const int lr0 = 4 * lane;
  int l[4], e[4], tot = 0;
  unsigned vbits = 0;
  int a[4];
  {
    const int4 q = *reinterpret_cast<const int4*>(soff + lr0);
    const int a4 = soff[lr0 + 4];
    a[0] = q.x, a[1] = q.y, a[2] = q.z, a[3] = q.w;
    vbits = (sbm[lr0 >> 5] >> (lr0 & 31)) & 15u;
    const int d[4] = {q.y - q.x, q.z - q.y, q.w - q.z, a4 - q.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const bool in = lr0 + k < NR;
      l[k] = !in ? 0 : (((vbits >> k) & 1u) ? min(max(d[k], 0), xc) : nl);  // R5 FirstX cap
      if (!in) vbits &= ~(1u << k);
      e[k] = tot;
      tot += l[k];
    }
  }
  const int incl = warp_incl_scan(tot, lane);
  const int L = incl - tot;
  const int T = __shfl_sync(0xffffffffu, incl, 31);
  const long long lb = base + L;
  store_quad(p.c.lengths + (int64_t)f * B + R0 + lr0, p.c.offsets + (int64_t)f * B + R0 + lr0, R0 + lr0, B, l, lb,
             e);
  if (f == p.c.n_sparse_out - 1 && rt == p.c.tiles_per_feature - 1 && lane == 31) {
    p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + T;  // total, R17
    if (base + T > p.c.values_cap) atomicExch(p.c.err, 1);
  }
  // change points: a producing row whose delta differs from the previous
  // row's, follows a row that emits nothing, or is a filled null
  int nc = 0;
  {
    int eff[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) eff[k] = ((vbits >> k) & 1u) ? a[k] - (L + e[k]) : kNullRow;
    int pe = __shfl_up_sync(0xffffffffu, eff[3], 1), pl = __shfl_up_sync(0xffffffffu, l[3], 1);
    if (lane == 0) pl = 0;
    unsigned cpm = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const bool c = l[k] > 0 && (pl == 0 || eff[k] != pe || eff[k] == kNullRow);
      cpm |= (c ? 1u : 0u) << k;
      pe = eff[k];
      pl = l[k];
    }
    const int cnt = __popc(cpm);
    const int ci = warp_incl_scan(cnt, lane);
    nc = __shfl_sync(0xffffffffu, ci, 31);
    int w = ci - cnt;
#pragma unroll
    for (int k = 0; k < 4; ++k)
      if ((cpm >> k) & 1u) cps[w++] = make_int2(L + e[k], eff[k]);
  }
  __syncwarp();
  const int64_t* val = p.val[src];
  int64_t* values = p.c.values;
  constexpr bool vi32 = I32;  // Cast: int32 values (RAP_OUT_VALUES_I32)
  const long long cap = p.c.values_cap;
  // hoisted: the window loop's stores go through a generic pointer that the
  // compiler cannot prove disjoint from the parameter block, so a p.c field
  // read inside the loop is reloaded per window (ncu: a generic 8-byte load
  // of p.c.itab was the top long-scoreboard stall of C4)
  const int64_t* const itab = p.c.itab;
  int64_t* ring = reinterpret_cast<int64_t*>(wscr + kMultiRing);  // [4][128]
  uint32_t masks = 0;
  const int nwin = (T + 127) >> 7;
  // cur: last change point at or before the window start; nxp: position of
  // the next one (INT_MAX: none) -- warp-uniform, kept in registers
  int cur = 0, nxp = nc > 1 ? cps[1].x : INT_MAX;
  auto issue = [&](int w) {
    const int eb = w * 128;
    while (nxp <= eb) {
      ++cur;
      nxp = cur + 1 < nc ? cps[cur + 1].x : INT_MAX;
    }
    const int d0 = cps[cur].y;
    int dd[4] = {d0, d0, d0, d0};
    const bool inner = nxp < eb + 128;  // a change point inside the window
    if (inner)
      for (int j = cur + 1; j < nc; ++j) {  // (few)
        const int2 c = cps[j];
        if (c.x >= eb + 128) break;
#pragma unroll
        for (int u = 0; u < 4; ++u) dd[u] = c.x <= eb + 32 * u + lane ? c.y : dd[u];
      }
    unsigned act = 0, full = 0;
    int64_t* slot = ring + (w & 3) * 128;
    if (eb + 128 <= T && !inner && d0 != kNullRow) {
      // one contiguous input run (the steady state): 4 copies off one address
      const int64_t* src = val + (eb + lane + d0);
#pragma unroll
      for (int u = 0; u < 4; ++u) cp_async8(slot + 32 * u + lane, src + 32 * u);
      act = full = 15u;
    } else {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int ee = eb + 32 * u + lane;
        const bool in = ee < T;
        const bool va = in && dd[u] != kNullRow;
        act |= (in ? 1u : 0u) << u;
        full |= (va ? 1u : 0u) << u;
        if (va)
          cp_async8(slot + 32 * u + lane, val + (ee + dd[u]));
        else
          slot[32 * u + lane] = fc.fill;
      }
    }
    masks = (masks & ~(0xffu << (8 * (w & 3)))) | ((act | (full << 4)) << (8 * (w & 3)));
  };
  for (int w = 0; w < kMultiDepth; ++w) {  // exactly kMultiDepth groups (some empty),
    if (w < nwin) issue(w);                  // so wait_group<kMultiDepth> below
    cp_async_commit();                       // always covers window w
  }
  for (int w = 0; w < nwin; ++w) {
    if (w + kMultiDepth < nwin) issue(w + kMultiDepth);
    cp_async_commit();  // (possibly empty) keeps one group per window
    cp_async_wait_group<kMultiDepth>();
    const unsigned mk = (masks >> (8 * (w & 3))) & 0xffu;
    const unsigned act = mk & 15u, full = mk >> 4;
    const int64_t* slot = ring + (w & 3) * 128;
    int64_t x[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) x[u] = slot[32 * u + lane];  // this lane's own copies
    canon_apply_n<4>(fc.q, itab, x, act, full);
    const long long pos0 = base + w * 128 + lane;
    if (act == 15u && pos0 + 96 < cap) {
#pragma unroll
      for (int u = 0; u < 4; ++u) st_val(values, vi32, pos0 + 32 * u, x[u]);
    } else {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const long long pos = pos0 + 32 * u;
        if (((act >> u) & 1u) && pos < cap) st_val(values, vi32, pos, x[u]);
      }
    }
  }
  cp_async_wait_all();
  __syncwarp();
  return T;
}

// Tile of any other SRC_SPARSE / SRC_DENSE_BUCKET chain (op interpreter).
template <class P>
__device__ __noinline__ long long value_tile_generic(const P& p, int f, int64_t rt, int lane, long long base) {
  const SProg& pg = p.c.sprogs[f];
  const DevOp* ops = prog_ops(pg, p.c.ops);
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rt * kTileRows;
  int64_t* offsets = p.c.offsets + (int64_t)f * B;
  int32_t* lengths = p.c.lengths + (int64_t)f * B;
  int64_t* values = p.c.values;
  const bool vi32 = p.c.vi32 != 0;  // Cast: int32 values (RAP_OUT_VALUES_I32)
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
#pragma unroll
  for (int g = 0; g < kGroups; ++g) {
    const int64_t row = r0 + 32 * g + lane;
    if (row < B) {
      __stcs(lengths + row, len[g]);
      st_cs64(offsets + row, base + gb[g] + lex[g]);
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
      if (len[g] == 1 && pos < cap) st_val(values, vi32, pos, v1[g]);
    }
    return run;
  }
  // general (multi-id rows): elements in output order, per row group
#pragma unroll 1
  for (int g = 0; g < kGroups; ++g)
    value_group_general(p, f, r0 + 32 * g, lane, len[g], st[g], lex[g], base + gb[g]);
  return run;
}

// Offsets and ids of sparse tile (f, rt) whose first id goes to
// values[base]; returns the tile's output length total.
template <class P>
__device__ __forceinline__ long long value_tile(const P& p, FeatCtx& fc, int64_t rt, int lane, long long base,
                                                int32_t* scr) {
  if (fc.kind == TK_CANON) return value_tile_canon(p, fc, rt, lane, base);
  if (fc.kind == TK_NGRAM_FAST) {
    if (!fc.ng_staged) ngram_stage(p, fc.f, scr, lane);
    fc.ng_staged = 1;
    const long long T = ngram_tile_fast(p, fc.f, rt, lane, base, scr);
    if (T >= 0) return T;
    fc.ng_staged = 0;  // the general path reuses the scratch
  }
  if (fc.kind != TK_GENERIC) return value_tile_ngram(p, fc.f, rt, lane, base, scr);
  return value_tile_generic(p, fc.f, rt, lane, base);
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
      if (pos < cap) st_val(p.c.values, p.c.vi32 != 0, pos, v);
    }
  }
}

// Output length total of the NGram tile starting at row r0 (R7 count
// max(0, sum of source lengths - n + 1), capped by FirstX): quad layout, 4
// rows per lane, every source's offsets requested before any is used.
// Output length total of the NGram tiles starting at rows r0 and r0 + 128
// (nt = 1 or 2) of a feature with k <= 4 sparse sources: all 2k quads in
// flight together.
template <class P>
__device__ __noinline__ long long ngram_tiles_len2(const P& p, const SProg& pg, int64_t r0, int nt, int lane) {
  const int64_t B = p.c.n_rows;
  const int k = pg.ng.k, n = pg.ng.n;
  const int64_t xo = pg.ch.xcap;
  Chain sc[4];
#pragma unroll
  for (int j = 0; j < 4; ++j)
    if (j < k) sc[j] = pg.src[j];
  Quad q[2][4];
#pragma unroll
  for (int t = 0; t < 2; ++t)
#pragma unroll
    for (int j = 0; j < 4; ++j)
      if (t < nt && j < k) {
        const int32_t* off = p.off[sc[j].src];
        q[t][j] = load_quad(off, p.svalid[sc[j].src], r0 + t * kTileRows, lane, B,
                            (reinterpret_cast<uintptr_t>(off) & 15) == 0);
      }
  int sum = 0;
#pragma unroll
  for (int t = 0; t < 2; ++t)
    if (t < nt) {
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const int64_t row = r0 + t * kTileRows + 4 * lane + kk;
        int tot = 0;
#pragma unroll
        for (int j = 0; j < 4; ++j)
          if (j < k) tot += quad_len(q[t][j], kk, lane, row, B, sc[j].xcap, sc[j].has_fill, sc[j].null_xcap);
        if (row < B) sum += (int32_t)min((int64_t)max(tot - n + 1, 0), xo);
      }
    }
  return warp_sum64(sum);
}

template <class P>
__device__ __noinline__ long long ngram_tile_len(const P& p, const SProg& pg, int64_t r0, int lane) {
  const int64_t B = p.c.n_rows;
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
  return warp_sum64(sum);
}

// Warp-cooperative copy of `bytes` (a multiple of 8) from global to shared.
__device__ __forceinline__ void warp_copy8(void* dst, const void* src, int bytes, int lane) {
  const long long* s8 = reinterpret_cast<const long long*>(src);
  long long* d8 = reinterpret_cast<long long*>(dst);
  for (int i = lane; i < (bytes >> 3); i += 32) d8[i] = __ldg(s8 + i);
}

struct NgParams {  // ngram_tile_fast parameters, staged in warp scratch
  Chain src[4];
  Canon scn[4];
  Canon post;
  NGramDesc ng;
  int64_t xcap;
};
static_assert(offsetof(NgParams, scn) == sizeof(Chain) * 4 && offsetof(NgParams, post) == offsetof(NgParams, scn) + sizeof(Canon) * 4 &&
                  offsetof(NgParams, ng) == offsetof(NgParams, post) + sizeof(Canon) && sizeof(Chain) % 8 == 0 &&
                  sizeof(Canon) % 8 == 0 && sizeof(NGramDesc) % 8 == 0,
              "NgParams is staged as one run of 8-byte words");
constexpr int kNgParamWords = align_up((int)sizeof(NgParams), 16) / 4;
constexpr int kNgStageOff = kTileRows + 4;  // staged offsets per source (129 used, 16-byte rows)
static_assert((kNgParamWords + 4 * kTileRows + 4 * kNgStageOff + 16) * 4 <= kWarpScr, "ngram_tile_fast scratch too large");

// Stage feature f's fast-NGram parameters into the warp scratch: every
// lane's loads in flight before any store.
template <class P>
__device__ __forceinline__ void ngram_stage(const P& p, int f, int32_t* scr, int lane) {
  const SProg& pg = p.c.sprogs[f];
  NgParams& G = *reinterpret_cast<NgParams*>(scr);
  constexpr int W1 = sizeof(G.src) / 8, W2 = sizeof(G.scn) / 8, W3 = sizeof(G.post) / 8, W4 = sizeof(G.ng) / 8;
  constexpr int WT = W1 + W2 + W3 + W4, PER = (WT + 31) / 32;
  long long r[PER];
#pragma unroll
  for (int i = 0; i < PER; ++i) {
    const int w = lane + 32 * i;
    const long long* src = w < W1 ? reinterpret_cast<const long long*>(pg.src) + w
                         : w < W1 + W2 ? reinterpret_cast<const long long*>(pg.src_cn) + (w - W1)
                         : w < W1 + W2 + W3 ? reinterpret_cast<const long long*>(&pg.cn) + (w - W1 - W2)
                                            : reinterpret_cast<const long long*>(&pg.ng) + (w - W1 - W2 - W3);
    if (w < WT) r[i] = __ldg(src);
  }
  long long* dst = reinterpret_cast<long long*>(&G);  // src, scn, post, ng are contiguous in NgParams
#pragma unroll
  for (int i = 0; i < PER; ++i)
    if (lane + 32 * i < WT) dst[lane + 32 * i] = r[i];
  if (lane == 0) G.xcap = pg.ch.xcap;
  __syncwarp();
}

// Fast NGram tile (R7) for k <= 4 canonical single-source chains when every
// row of every source has at most one id and at most n ids in total: then a
// row has one window (exactly n ids) or none, and its hash is the chain over
// the present ids in source order.  Quad layout (4 rows per lane); all
// sources' offsets, then all their ids, are in flight together.  Returns
// the tile's output length total, or -1 with nothing written when the tile
// is not eligible.
template <class P>
__device__ __noinline__ long long ngram_tile_fast(const P& p, int f, int64_t rt, int lane, long long base,
                                                 int32_t* scr) {
  trace_clk(p.c, 13, 0);
  // parameters: staged in warp-private shared memory by ngram_stage (no lazy
  // global reads on the dependent path); per-(source, row) id positions after
  const NgParams& G = *reinterpret_cast<const NgParams*>(scr);
  int32_t* pos = scr + kNgParamWords;  // [4][kTileRows]: child index, -1 = fill, -2 = absent
  // every source's offsets / validity words staged with cp.async (no quads
  // held in registers): [4][kNgStageOff] int32 then [4][4] u32 after pos
  int32_t* soff = pos + 4 * kTileRows;
  uint32_t* sbm = reinterpret_cast<uint32_t*>(soff + 4 * kNgStageOff);
  const int k = G.ng.k, n = G.ng.n;
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rt * kTileRows;
  const int64_t row = r0 + 4 * lane;
  const int NR = (int)min((int64_t)kTileRows, B - r0);
#pragma unroll
  for (int j = 0; j < 4; ++j)
    if (j < k) stage_offsets(p.off[G.src[j].src], p.svalid[G.src[j].src], r0, NR, soff + j * kNgStageOff, sbm + 4 * j, lane);
  cp_async_wait_all();
  __syncwarp();
  // per (source, row) output lengths of the lane's 4 rows, 4 bits each
  int pn[4] = {0, 0, 0, 0};
  unsigned l1 = 0, fullm = 0;  // bit 4j+kk: source j of row kk has one id / is valid
  bool ok = true;
#pragma unroll
  for (int j = 0; j < 4; ++j)
    if (j < k) {
      const Chain& sc = G.src[j];
      const int xc = (int)min(sc.xcap, (int64_t)INT32_MAX);
      const int nl = sc.has_fill ? (int)min((int64_t)1, sc.null_xcap) : 0;  // R10 / R14
      const int32_t* so = soff + j * kNgStageOff;
      const int lr0 = 4 * lane;
      const int4 a = *reinterpret_cast<const int4*>(so + lr0);  // 16-byte aligned rows
      const int a4 = so[lr0 + 4];
      const unsigned vb = (sbm[4 * j + (lr0 >> 5)] >> (lr0 & 31)) & 15u;
      const int d[4] = {a.y - a.x, a.z - a.y, a.w - a.z, a4 - a.w};
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const bool in = lr0 + kk < NR;
        const bool fu = in && ((vb >> kk) & 1u);
        const int l = !in ? 0 : (fu ? min(max(d[kk], 0), xc) : nl);  // R5 FirstX cap
        ok &= l <= 1;
        pn[kk] += l;
        l1 |= (l == 1 ? 1u : 0u) << (4 * j + kk);
        fullm |= (fu ? 1u : 0u) << (4 * j + kk);
      }
    }
#pragma unroll
  for (int kk = 0; kk < 4; ++kk) ok &= pn[kk] <= n;
  if (!__all_sync(0xffffffffu, ok)) {
    __syncwarp();
    return -1;
  }
  int32_t l[4], e[4];
  int tot = 0;
#pragma unroll
  for (int kk = 0; kk < 4; ++kk) {
    l[kk] = (row + kk < B && pn[kk] == n) ? (int32_t)min((int64_t)1, G.xcap) : 0;
    e[kk] = tot;
    tot += l[kk];
  }
  // presence (bit 4j+kk) and id positions of every (source, row)
  unsigned pres = 0, full = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j)
    if (j < k) {
      int a[4];
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const unsigned bit = 1u << (4 * j + kk);
        const bool pr = l[kk] == 1 && (l1 & bit);
        const bool fu = fullm & bit;
        pres |= pr ? bit : 0u;
        full |= fu ? bit : 0u;
        a[kk] = pr ? (fu ? soff[j * kNgStageOff + 4 * lane + kk] : -1) : -2;
      }
      *reinterpret_cast<int4*>(pos + j * kTileRows + 4 * lane) = make_int4(a[0], a[1], a[2], a[3]);
    }
  const int incl = warp_incl_scan(tot, lane);
  const int L = incl - tot;
  const int T = __shfl_sync(0xffffffffu, incl, 31);
  const long long lb = base + L;
  store_quad(p.c.lengths + (int64_t)f * B + row, p.c.offsets + (int64_t)f * B + row, row, B, l, lb, e);
  const int64_t* itab = p.c.itab;
  uint64_t h[4];
#pragma unroll
  for (int kk = 0; kk < 4; ++kk) h[kk] = G.ng.hsalt;  // R7: h = H(salt); h = H(h ^ c[q])
  // sources in order, the next source's ids in flight while this one runs
  // its canonical pipeline (R3-R8) and feeds the window hash
  int64_t vn[4];
  auto load_src = [&](int j, int64_t (&v)[4]) {
    const int4 a = *reinterpret_cast<const int4*>(pos + j * kTileRows + 4 * lane);
    const int64_t* val = p.val[G.src[j].src];
    const int64_t fill = G.src[j].fill;
    v[0] = a.x >= 0 ? __ldg(val + a.x) : fill;
    v[1] = a.y >= 0 ? __ldg(val + a.y) : fill;
    v[2] = a.z >= 0 ? __ldg(val + a.z) : fill;
    v[3] = a.w >= 0 ? __ldg(val + a.w) : fill;
  };
  load_src(0, vn);
  trace_clk(p.c, 14, vn[0] + vn[3]);
#pragma unroll 1
  for (int j = 0; j < k; ++j) {
    int64_t v[4] = {vn[0], vn[1], vn[2], vn[3]};
    if (j + 1 < k) load_src(j + 1, vn);
    const unsigned pj = (pres >> (4 * j)) & 15u, fj = (full >> (4 * j)) & 15u;
    canon_apply_n<4>(G.scn[j], itab, v, pj, fj);
#pragma unroll
    for (int kk = 0; kk < 4; ++kk)
      if ((pj >> kk) & 1u) h[kk] = splitmix_H(h[kk] ^ (uint64_t)v[kk]);
  }
  int64_t o[4];
  unsigned act = 0;
#pragma unroll
  for (int kk = 0; kk < 4; ++kk) {
    o[kk] = (int64_t)reduce_M(h[kk], G.ng.M);
    act |= (l[kk] == 1 ? 1u : 0u) << kk;
  }
  canon_apply_n<4>(G.post, itab, o, act, 15u);
  const long long cap = p.c.values_cap;
#pragma unroll
  for (int kk = 0; kk < 4; ++kk)
    if (((act >> kk) & 1u) && lb + e[kk] < cap) st_val(p.c.values, p.c.vi32 != 0, lb + e[kk], o[kk]);
  if (f == p.c.n_sparse_out - 1 && rt == p.c.tiles_per_feature - 1 && lane == 31) {
    p.c.offsets[(int64_t)p.c.n_sparse_out * B] = base + T;  // total, R17
    if (base + T > cap) atomicExch(p.c.err, 1);
  }
  trace_clk(p.c, 15, 0);
  __syncwarp();
  return T;
}

// NGram feature tile (R7): per row the k source lists, windows over their
// concatenation.
template <class P>
__device__ __noinline__ long long value_tile_ngram(const P& p, int f, int64_t rt, int lane, long long base,
                                                   int32_t* scr) {
  const SProg& pg = p.c.sprogs[f];
  const DevOp* ops = prog_ops(pg, p.c.ops);
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rt * kTileRows;
  int64_t* offsets = p.c.offsets + (int64_t)f * B;
  int32_t* lengths = p.c.lengths + (int64_t)f * B;
  int64_t* values = p.c.values;
  const bool vi32 = p.c.vi32 != 0;  // Cast: int32 values (RAP_OUT_VALUES_I32)
  const long long cap = p.c.values_cap;

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
      __stcs(lengths + row, len);
      st_cs64(offsets + row, run + lx);
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
          ev_s[c * 32 + lane] = canon1(qc, itab, ev_s[c * 32 + lane], st_s[c * 32 + lane] >= 0);
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
        const int64_t v = canon1(qp, itab, (int64_t)reduce_M(h, pg.ng.M), true);
        const long long pos = run + lx + j;
        if (pos < cap) st_val(values, vi32, pos, v);
      }
    } else if (__all_sync(0xffffffffu, len <= 1)) {
      if (len == 1) {
        const long long pos = run + lx;
        const int64_t v = ngram_window(p, pg, ops, st_s + lane, sl_s + lane, 32, row, 0);
        if (pos < cap) st_val(values, vi32, pos, v);
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
          if (pos < cap) st_val(values, vi32, pos, v);
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
  return run - base;
}

// ----------------------------------------------------------------------------
// Phase L: output length total of sparse tile (f, rt) (closed forms R5, R7,
// R10, R14 from the Arrow offsets and validity words only).
template <class P>
__device__ __noinline__ long long tile_total(const P& p, int f, int64_t rt, int lane) {
  const int64_t B = p.c.n_rows;
  const int64_t r0 = rt * kTileRows;
  const SProg& pg = p.c.sprogs[f];
  if (pg.ch.src_kind == SRC_NGRAM) return ngram_tile_len(p, pg, r0, lane);
  return min((int64_t)kTileRows, B - r0) * min((int64_t)1, pg.ch.xcap);  // R4: dense bucket, 1 id per row
}

__device__ __forceinline__ long long block_sum(long long v, long long* red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  v = warp_sum64(v);
  __syncthreads();
  if (lane == 0) red[warp] = v;
  __syncthreads();
  long long t = 0;
#pragma unroll
  for (int j = 0; j < kWarps; ++j) t += red[j];
  return t;
}

#ifndef RAP_MIN_CTAS
#define RAP_MIN_CTAS 3  // 85 registers: the fastest of 2/3/4 on the C2 graph (profiles/README.md)
#endif
template <int MD, int MS>
__global__ void __launch_bounds__(kThreads, RAP_MIN_CTAS) rap_fused_kernel(const __grid_constant__ KParams<MD, MS> p) {
  unsigned char* const smem = rap_dyn_smem;
  __shared__ CtaState cs;
  __shared__ long long s_slots[kWarps];
  __shared__ long long s_red[kWarps];
  __shared__ int s_last;
  __shared__ FeatCtx s_fc[kWarps];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // The epoch load is consumed only when the aggregate is published, so its
  // latency hides under the length pass.  Ranks are block indices: the
  // launch is cooperative, so every CTA is resident and a CTA waits only on
  // resident predecessors.
  const unsigned long long epoch = ld_relaxed(p.c.sched + 1);
  // chained launch (rap_output.flags & RAP_OUT_CHAIN): offsets[0] already
  // holds the running total of the launch before this one into the same
  // buffer; every offset and value position of this launch starts there (the
  // first tile rewrites offsets[0] with the same value)
  const long long chain0 = p.c.chain ? (long long)__ldg(p.c.offsets) : 0ll;
#ifdef RAP_TRACE_CLK
  if (tid < 24) s_clk[tid] = 0;
#endif
  if (tid == 0) {
    mbar_init(&cs.bar, 1);
    cs.phase = 0;
    cs.dgroup = -1;
    // no sparse outputs: the offsets array is the single total 0 (R17)
    if (blockIdx.x == 0 && p.c.n_sparse_out == 0 && !p.c.chain && p.c.offsets) p.c.offsets[0] = 0;
  }
  trace_stamp(p.c, 0);
  const int rank = blockIdx.x;
  if (p.c.trace != nullptr && tid == 0 && (int64_t)blockIdx.x < p.c.trace_cap) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    p.c.trace[(int64_t)blockIdx.x * kTracePts + 6] = smid;
    p.c.trace[(int64_t)blockIdx.x * kTracePts + 7] = (unsigned long long)rank;
  }
  const int64_t S = p.c.n_sparse_tiles, T = p.c.tiles_per_feature;
  // my sparse tiles [s0, s1) and my warp's [w0, w1) (host per-warp partition)
  // (clamped to [0, S]: a partition of another batch shape -- a misuse of a
  // captured graph, rap.h -- can leave tiles unwritten but never leave S)
  const int64_t s0 = clamp_tile(__ldg(p.c.part + rank * kWarps), 0, S);
  const int64_t s1 = clamp_tile(__ldg(p.c.part + (rank + 1) * kWarps), s0, S);
  const int64_t w0 = clamp_tile(__ldg(p.c.part + rank * kWarps + warp), 0, S);
  const int64_t w1 = clamp_tile(__ldg(p.c.part + rank * kWarps + warp + 1), w0, S);
  unsigned char* wscr = smem + warp * kWarpScr;  // warp-private region (sparse phases)
  int32_t* scr = reinterpret_cast<int32_t*>(wscr);
  if (p.c.trace != nullptr && tid == 0 && (int64_t)blockIdx.x < p.c.trace_cap)
    p.c.trace[(int64_t)blockIdx.x * kTracePts + 5] = (unsigned long long)(s0 | ((s1 - s0) << 32));

  // (L) output length total of my warp's sub-range -> CTA aggregate
  long long mine = 0, part = 0;  // warp-uniform / per-lane partial totals
  trace_clk(p.c, 21, 0);
  // per-feature dispatch state in warp-private shared memory (not registers:
  // it is live across the whole tile loop)
  FeatCtx& fc = s_fc[warp];
  if (lane == 0) fc.f = -1;
  __syncwarp();
  {
    const int64_t B = p.c.n_rows;
    int fcur = 0;
    int64_t fend = -1;
    for (int64_t t = w0; t < w1;) {
      if (t >= fend) {  // feature boundary: one 64-bit division per feature, not per tile
        fcur = (int)((uint64_t)t / (uint64_t)T);
        fend = (int64_t)(fcur + 1) * T;
      }
      const int f = fcur;
      // every lane reads the cached feature before any lane rewrites it
      // (independent thread scheduling: racecheck WAR otherwise)
      const bool reload = f != fc.f;
      __syncwarp();
      if (reload) load_ctx(p, f, fc);  // ends with __syncwarp
      const int64_t tend = min(w1, (int64_t)(f + 1) * T);
      if (fc.sk == SRC_SPARSE) {
        // kLChunkTiles tiles' offsets and validity words staged per round
        const int32_t* off = p.off[fc.src];
        const uint32_t* bm = p.svalid[fc.src];
        int32_t* soff = reinterpret_cast<int32_t*>(wscr + kLStageOff);
        uint32_t* sbm = reinterpret_cast<uint32_t*>(wscr + kLStageBm);
        const int64_t xcap = fc.xcap, null_xcap = fc.null_xcap;
        const int has_fill = fc.has_fill;
        while (t < tend) {
          const int nt = (int)min((int64_t)kLChunkTiles, tend - t);
          const int64_t R0 = (t - (int64_t)f * T) * kTileRows;
          const int NR = (int)min((int64_t)nt * kTileRows, B - R0);
          stage_offsets(off, bm, R0, NR, soff, sbm, lane);
          cp_async_wait_all();
          __syncwarp();
          const int xc = (int)min(xcap, (int64_t)INT32_MAX);
          const int nl = has_fill ? (int)min((int64_t)1, null_xcap) : 0;  // R10 / R14
          for (int lr0 = 4 * lane; lr0 < NR; lr0 += 128) {  // 4 rows per lane per step
            const int4 a = *reinterpret_cast<const int4*>(soff + lr0);
            const int a4 = soff[lr0 + 4];
            const unsigned vb = (sbm[lr0 >> 5] >> (lr0 & 31)) & 15u;
            const int d[4] = {a.y - a.x, a.z - a.y, a.w - a.z, a4 - a.w};
#pragma unroll
            for (int k = 0; k < 4; ++k)
              if (lr0 + k < NR) part += ((vb >> k) & 1u) ? min(max(d[k], 0), xc) : nl;  // R5 FirstX cap
          }
          __syncwarp();
          t += nt;
        }
      } else if (fc.kind == TK_NGRAM_FAST) {
        const SProg& pg = p.c.sprogs[f];
        while (t < tend) {
          const int nt = (int)min((int64_t)2, tend - t);
          mine += ngram_tiles_len2(p, pg, (t - (int64_t)f * T) * kTileRows, nt, lane);  // warp-uniform
          t += nt;
        }
      } else {
        for (; t < tend; ++t) mine += tile_total(p, f, t - (int64_t)f * T, lane);  // warp-uniform
      }
    }
  }
  mine += warp_sum64(part);
  trace_clk(p.c, 22, mine);
  if (lane == 0) s_slots[warp] = mine;
  const long long agg = block_sum(lane == 0 ? mine : 0ll, s_red);
  trace_clk(p.c, 23, agg);
  const unsigned long long tag = epoch + 1ull;
  if (tid == 0) st_relaxed(p.c.agg + rank, (tag << kEpochShift) | (unsigned long long)agg);
  trace_stamp(p.c, 1);

  // (D) my dense blocks, round robin over the ranks (independent of the
  // scan: they hide the wait below)
#ifdef RAP_DBG_SKIP_D
  if (false)
#endif
  for (int64_t d = rank; d < p.c.n_dense_tiles; d += gridDim.x) {
    const uint32_t gi = (uint32_t)d % (uint32_t)p.c.n_groups;
    dense_block(p, (int)gi, (int64_t)((uint32_t)d / (uint32_t)p.c.n_groups), 0, cs);
    __syncthreads();
  }
  trace_stamp(p.c, 2);

  if (s1 > s0) {
    // (W) base of my range = sum of the aggregates of the CTAs ranked before
    // me; all of them were resident before I started
    // warp 0 polls (32 lanes, backoff), so waiting CTAs do not flood the
    // L2 slices that hold the aggregate words
    long long pre = 0;
    if (warp == 0) {
      for (int j0 = 0; j0 < rank; j0 += 32 * 8) {
        unsigned long long w[8];
        bool ready = false;
        int ns = 128;
        while (!ready) {
          ready = true;
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            const int j = j0 + 32 * u + lane;
            w[u] = j < rank ? ld_relaxed(p.c.agg + j) : (tag << kEpochShift);
            ready &= (w[u] >> kEpochShift) == tag;
          }
          ready = __all_sync(0xffffffffu, ready);
          if (!ready) {
            __nanosleep(ns);
            ns = min(ns * 2, 2048);
          }
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) pre += (long long)(w[u] & kValueMask);
      }
    }
    const long long base = block_sum(pre, s_red) + chain0;
    trace_stamp(p.c, 3);

    // (V) offsets and ids of my warp's tiles, in scan order
    if (lane == 0) fc.f = -1;
    __syncwarp();
    long long run = base;
    for (int j = 0; j < warp; ++j) run += s_slots[j];
#ifdef RAP_DBG_SKIP_V
    if (false)
#endif
    int fcur = 0;
    int64_t fend = -1;
    for (int64_t t = w0; t < w1;) {
      if (t >= fend) {  // feature boundary: one 64-bit division per feature, not per tile
        fcur = (int)((uint64_t)t / (uint64_t)T);
        fend = (int64_t)(fcur + 1) * T;
      }
      const int f = fcur;
      const bool reload = f != fc.f;
      __syncwarp();
      if (reload) load_ctx(p, f, fc);  // ends with __syncwarp
      if (fc.kind == TK_CANON) {
        const int nt = (int)min((int64_t)kVChunkTiles, min(w1, (int64_t)(f + 1) * T) - t);
        const long long got = value_chunk_canon(p, fc, t - (int64_t)f * T, nt, lane, run, wscr);
        if (got >= 0) {
          run += got;
          t += nt;
          continue;
        }
        // multi-id rows: element-parallel tiles
        for (int j = 0; j < nt; ++j)
          run += p.c.vi32 ? value_tile_multi<true>(p, fc, t + j - (int64_t)f * T, lane, run, wscr)
                          : value_tile_multi<false>(p, fc, t + j - (int64_t)f * T, lane, run, wscr);
        t += nt;
        continue;
      }
      run += value_tile(p, fc, t - (int64_t)f * T, lane, run, scr);
      ++t;
    }
  }
  trace_stamp(p.c, 4);

#ifdef RAP_TRACE_CLK
  __syncthreads();
  if (p.c.trace != nullptr && tid >= 8 && tid < 24 && (int64_t)blockIdx.x < p.c.trace_cap)
    p.c.trace[(int64_t)blockIdx.x * kTracePts + tid] = s_clk[tid];
#endif
  // The last CTA out resets the rank counter and advances the epoch of the
  // aggregate words (clearing them when the 20-bit epoch wraps), so launch
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
      for (int64_t i = tid; i < kMaxCtas; i += kThreads) p.c.agg[i] = 0ull;
    __syncthreads();
    if (tid == 0) {
      p.c.sched[0] = 0ull;
      p.c.sched[1] = wrap ? 0ull : epoch + 1ull;
      __threadfence();
    }
  }
}

template <int MD, int MS>
static int launch_t(const Common& c, const LaunchRaw& raw, int grid, int smem, cudaStream_t st) {
  static_assert(sizeof(KParams<MD, MS>) <= 32000, "kernel parameter block too large");
  const int rc = ensure_dyn_smem(reinterpret_cast<const void*>(rap_fused_kernel<MD, MS>), smem);
  if (rc != 0) return rc;
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
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;  // all CTAs co-resident (the scan waits on predecessors)
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
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

int ensure_dyn_smem(const void* kernel, int smem) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, int> set;  // (kernel, device) -> attribute value
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return (int)e;
  std::lock_guard<std::mutex> lk(mu);
  int& cur = set[std::make_pair(kernel, dev)];
  if (cur >= smem) return 0;
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return (int)e;
  cur = smem;
  return 0;
}

int fused_occupancy(int smem_bytes, int n_dense, int n_sparse, int* ctas_per_sm) {
  const void* k = n_dense <= 32 && n_sparse <= 64 ? reinterpret_cast<const void*>(rap_fused_kernel<32, 64>)
                                                  : reinterpret_cast<const void*>(rap_fused_kernel<128, 1024>);
  const int rc = ensure_dyn_smem(k, smem_bytes);
  if (rc != 0) return rc;
  return (int)cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, k, kThreads, smem_bytes);
}

}  // namespace rapk

// ----------------------------------------------------------------------------
// rap_jagged_append (include/rap.h): a received residual piece continues a
// chained jagged output.  Grid-stride copy; the running total
// T = dst_offsets[0] is a device value (written by the preceding launch).
namespace rapk {

__global__ void __launch_bounds__(256) jagged_append_kernel(const int32_t* __restrict__ len,
                                                            const int64_t* __restrict__ so,
                                                            const int64_t* __restrict__ val, int64_t n,
                                                            int32_t* __restrict__ dl, int64_t* dof,
                                                            int64_t* __restrict__ dv, int64_t cap) {
  const long long T = *reinterpret_cast<volatile const long long*>(dof);
  const int64_t s0 = so[0];
  const int64_t nv = so[n] - s0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < max(n, nv); i += stride) {
    if (i < n) {
      dl[i] = len[i];
      dof[i + 1] = T + (so[i + 1] - s0);
    }
    if (i < nv && T + i < cap) dv[T + i] = val[s0 + i];
  }
}

// Exact-size D2H of a jagged output's values (rap_preprocess_host*): the
// total is the device value *total (offsets[F * B]); the kernel writes
// values[0, total) straight into pinned (device-mapped) host memory, so no
// host sync is needed to learn the count and no padding crosses PCIe.
__global__ void __launch_bounds__(256) values_to_host_kernel(const int64_t* __restrict__ src,
                                                             const int64_t* __restrict__ total, int64_t cap,
                                                             int64_t* __restrict__ dst) {
  const int64_t n = min(*total, cap);
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  // 16-byte moves (both buffers come from 256-byte aligned allocations)
  const int64_t n2 = n >> 1;
  const longlong2* s2 = reinterpret_cast<const longlong2*>(src);
  longlong2* d2 = reinterpret_cast<longlong2*>(dst);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n2; i += stride) d2[i] = s2[i];
  if ((n & 1) && blockIdx.x == 0 && threadIdx.x == 0) dst[n - 1] = src[n - 1];
}

int launch_values_to_host(const int64_t* src, const int64_t* total, int64_t cap, int64_t* dst, void* stream) {
  const int64_t blocks = min((cap / 2 + 255) / 256, (int64_t)148 * 4);
  values_to_host_kernel<<<(unsigned)max(blocks, (int64_t)1), 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(
      src, total, cap, dst);
  return (int)cudaGetLastError();
}

// Batched H2D of a host batch's columns (rap_preprocess_host*): every column
// lives in pinned (device-mapped) host memory, so one launch reads all of them
// across PCIe into their staging buffers.  One copy engine transfer per column
// (~100 for C2) costs ~8 us of engine time each and queues behind the other
// stream's D2H; the SMs' reads overlap it.  A block moves one 32 KB chunk of
// one copy; units are the widest of 16 / 8 / 4 / 1 bytes both ends allow.
constexpr int kGatherMax = 192;
constexpr int64_t kGatherChunk = 32768;
struct GatherCopy {
  const void* src;
  void* dst;
  int64_t bytes;
  int64_t blk0;  // first block of this copy
};
struct GatherParams {
  int n;
  GatherCopy c[kGatherMax];
};

template <typename T>
__device__ __forceinline__ void gather_chunk(const GatherCopy& c, int64_t b0, int64_t b1) {
  const T* __restrict__ s = static_cast<const T*>(c.src);
  T* __restrict__ d = static_cast<T*>(c.dst);
  const int64_t u0 = b0 / (int64_t)sizeof(T), u1 = b1 / (int64_t)sizeof(T);
  for (int64_t u = u0 + threadIdx.x; u < u1; u += 8 * 256) {
    T v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (u + k * 256 < u1) v[k] = s[u + k * 256];  // all loads in flight before the stores
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (u + k * 256 < u1) d[u + k * 256] = v[k];
  }
  const int64_t t0 = u1 * (int64_t)sizeof(T);  // bytes past the last whole unit
  if (threadIdx.x < b1 - t0)
    static_cast<char*>(c.dst)[t0 + threadIdx.x] = static_cast<const char*>(c.src)[t0 + threadIdx.x];
}

__global__ void __launch_bounds__(256) gather_h2d_kernel(const __grid_constant__ GatherParams p) {
  int lo = 0, hi = p.n - 1;  // the copy this block belongs to: last blk0 <= blockIdx.x
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (p.c[mid].blk0 <= (int64_t)blockIdx.x) lo = mid;
    else hi = mid - 1;
  }
  const GatherCopy& c = p.c[lo];
  const int64_t b0 = ((int64_t)blockIdx.x - c.blk0) * kGatherChunk;
  const int64_t b1 = min(c.bytes, b0 + kGatherChunk);
  const uintptr_t a = reinterpret_cast<uintptr_t>(c.src) | reinterpret_cast<uintptr_t>(c.dst);
  if ((a & 15) == 0) gather_chunk<int4>(c, b0, b1);
  else if ((a & 7) == 0) gather_chunk<long long>(c, b0, b1);
  else if ((a & 3) == 0) gather_chunk<int>(c, b0, b1);
  else gather_chunk<char>(c, b0, b1);
}

int launch_gather_h2d(const void* const* src, void* const* dst, const int64_t* bytes, int n, void* stream) {
  for (int i0 = 0; i0 < n; i0 += kGatherMax) {
    GatherParams p;
    p.n = 0;
    int64_t blocks = 0;
    for (int i = i0; i < n && i < i0 + kGatherMax; ++i) {
      if (bytes[i] <= 0) continue;
      p.c[p.n++] = GatherCopy{src[i], dst[i], bytes[i], blocks};
      blocks += (bytes[i] + kGatherChunk - 1) / kGatherChunk;
    }
    if (!blocks) continue;
    gather_h2d_kernel<<<(unsigned)blocks, 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(p);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return (int)e;
  }
  return 0;
}

int launch_jagged_append(const int32_t* len, const int64_t* so, const int64_t* val, int64_t n, int64_t vb, int32_t* dl,
                         int64_t* dof, int64_t* dv, int64_t cap, void* stream) {
  const int64_t work = max(n, vb);
  const int64_t blocks = min((work + 255) / 256, (int64_t)148 * 8);
  jagged_append_kernel<<<(unsigned)max(blocks, (int64_t)1), 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(
      len, so, val, n, dl, dof, dv, cap);
  return (int)cudaGetLastError();
}

}  // namespace rapk
