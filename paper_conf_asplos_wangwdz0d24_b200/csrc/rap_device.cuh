// rap_device.cuh — device helpers shared by the two fused kernels
// (rap_kernel.cu: tiled kernel; rap_rows.cu: row-block kernel).  Product
// code only; nothing here is shared with oracle/.  Operator semantics:
// DESIGN.md §3 readings R1-R20.
#pragma once
#ifndef __CUDACC_RTC__
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>
#endif

#include "rap_internal.h"

namespace rapk {

// The kernels' dynamic shared memory (one array per kernel launch; every
// extern __shared__ declaration names its start).
extern __shared__ __align__(128) unsigned char rap_dyn_smem[];

constexpr int kWarps = kThreads / 32;
__host__ __device__ constexpr int align_up(int x, int a) { return (x + a - 1) / a * a; }

// ----------------------------------------------------------------------------
// Scalar helpers.

__device__ __forceinline__ uint64_t reduce_M(uint64_t h, int64_t M) {  // R2: floor(h * M / 2^64)
  if (((uint64_t)M >> 32) == 0) {
    // M < 2^32 (every table size here): floor((hi*M + floor(lo*M / 2^32)) / 2^32), exact
    const uint64_t m = (uint64_t)M;
    const uint64_t t = (uint64_t)(uint32_t)(h >> 32) * m + (((uint64_t)(uint32_t)h * m) >> 32);
    return t >> 32;
  }
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

// cp.async (LDGSTS): global -> shared without a register round trip.
__device__ __forceinline__ void cp_async4(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async8(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait_group() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

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

// #{i : b[i] <= x} over sorted int64 b[0..m) with a sample table
// smp[i] = b[8i + 7] (i < m / 8): a binary search over the samples (a small
// table, L1-resident) finds the first block whose last border exceeds x, then
// the block's <= 8 borders are read in one burst (R4; same result as
// upper_bound).
__device__ __forceinline__ int64_t upper_bound_s8(const int64_t* b, int m, const int64_t* smp, int ns, int64_t x) {
  int lo = 0, n = ns;
  while (n > 0) {
    const int half = n >> 1;
    if (__ldg(smp + lo + half) <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  const int base = lo * 8;
  const int rem = min(8, m - base);
  int cnt = 0;
  if (rem == 8 && (reinterpret_cast<uintptr_t>(b + base) & 15) == 0) {
    const longlong2* q = reinterpret_cast<const longlong2*>(b + base);
    const longlong2 a0 = __ldg(q), a1 = __ldg(q + 1), a2 = __ldg(q + 2), a3 = __ldg(q + 3);
    cnt = (a0.x <= x) + (a0.y <= x) + (a1.x <= x) + (a1.y <= x) + (a2.x <= x) + (a2.y <= x) + (a3.x <= x) + (a3.y <= x);
  } else {
    for (int i = 0; i < rem; ++i) cnt += __ldg(b + base + i) <= x;
  }
  return base + cnt;
}

// Count of values <= x among 8 int64 at p (16-byte aligned), one burst.
__device__ __forceinline__ int count_le8(const int64_t* p, int64_t x) {
  const longlong2* q = reinterpret_cast<const longlong2*>(p);
  const longlong2 a0 = __ldg(q), a1 = __ldg(q + 1), a2 = __ldg(q + 2), a3 = __ldg(q + 3);
  return (a0.x <= x) + (a0.y <= x) + (a1.x <= x) + (a1.y <= x) + (a2.x <= x) + (a2.y <= x) + (a3.x <= x) + (a3.y <= x);
}

// #{i : b[i] <= x} over sorted int64 b[0..m), m a multiple of 64, given
// level-0 index j0 = #{blocks of 64 whose last border <= x} (the generated
// code computes it from immediates): then the 8 sub-block maxima of block j0
// (smp8[8 j0 .. 8 j0 + 8), smp8[i] = b[8 i + 7]) and the 8 borders of the
// chosen sub-block, two bursts (R4; same result as upper_bound).
// Same search over tables staged in shared memory (the generated kernel
// copies a plan's Bucketize borders and sub-block maxima there at launch).
__device__ __forceinline__ int count_le8_s(const int64_t* p, int64_t x) {
  const longlong2* q = reinterpret_cast<const longlong2*>(p);
  const longlong2 a0 = q[0], a1 = q[1], a2 = q[2], a3 = q[3];
  return (a0.x <= x) + (a0.y <= x) + (a1.x <= x) + (a1.y <= x) + (a2.x <= x) + (a2.y <= x) + (a3.x <= x) + (a3.y <= x);
}
__device__ __forceinline__ int64_t upper_bound_64s(const int64_t* b, int m, const int64_t* smp8, int j0, int64_t x) {
  const int nb = m >> 6;
  const int jc = min(j0, nb - 1);
  const int j1 = 8 * jc + min(count_le8_s(smp8 + 8 * jc, x), 7);
  const int64_t r = (int64_t)j1 * 8 + count_le8_s(b + 8 * j1, x);
  return j0 >= nb ? (int64_t)m : r;
}
// Sub-block maxima in shared memory, borders in global.
__device__ __forceinline__ int64_t upper_bound_64h(const int64_t* b, int m, const int64_t* smp8, int j0, int64_t x) {
  const int nb = m >> 6;
  const int jc = min(j0, nb - 1);
  const int j1 = 8 * jc + min(count_le8_s(smp8 + 8 * jc, x), 7);
  const int64_t r = (int64_t)j1 * 8 + count_le8(b + 8 * j1, x);
  return j0 >= nb ? (int64_t)m : r;
}
__device__ __forceinline__ int64_t upper_bound_64(const int64_t* b, int m, const int64_t* smp8, int j0, int64_t x) {
  // branch-free: the loads stay in range, the selects pick the answer
  const int nb = m >> 6;
  const int jc = min(j0, nb - 1);
  const int j1 = 8 * jc + min(count_le8(smp8 + 8 * jc, x), 7);
  const int64_t r = (int64_t)j1 * 8 + count_le8(b + 8 * j1, x);
  return j0 >= nb ? (int64_t)m : r;
}

// MapId (R8) whose first probe kv0 = table slot of x was loaded ahead (no
// INT64_MIN key; x may be INT64_MIN only if the table misses it).
__device__ __forceinline__ int64_t map_lookup_from(const int64_t* itab, int64_t a, int m, int64_t dflt, int64_t x,
                                                   longlong2 kv) {
  if (x == INT64_MIN) return dflt;
  const longlong2* t = reinterpret_cast<const longlong2*>(itab + a);
  const uint32_t mask = (1u << m) - 1u;
  uint32_t i = (uint32_t)(((uint64_t)x * 0x9E3779B97F4A7C15ull) >> (64 - m));
  while (true) {
    if (kv.x == x) return kv.y;
    if (kv.x == INT64_MIN) return dflt;
    i = (i + 1) & mask;
    kv = __ldg(t + i);
  }
}
// The first two probes of x (slots i and i + 1 of the linear-probing table),
// loaded ahead together: a lookup resolves without a dependent load unless
// both slots hold other keys (load <= 1/2: rare).
struct MapProbe2 {
  longlong2 a, b;
};
__device__ __forceinline__ MapProbe2 map_first_probe2(const int64_t* itab, int64_t a, int m, int64_t x) {
  const longlong2* t = reinterpret_cast<const longlong2*>(itab + a);
  const uint32_t mask = (1u << m) - 1u;
  const uint32_t i = (uint32_t)(((uint64_t)x * 0x9E3779B97F4A7C15ull) >> (64 - m));
  MapProbe2 r;
  r.a = __ldg(t + i);
  r.b = __ldg(t + ((i + 1u) & mask));
  return r;
}
__device__ __forceinline__ int64_t map_lookup_from2(const int64_t* itab, int64_t a, int m, int64_t dflt, int64_t x,
                                                    MapProbe2 kv) {
  if (x == INT64_MIN) return dflt;
  if (kv.a.x == x) return kv.a.y;
  if (kv.a.x == INT64_MIN) return dflt;
  if (kv.b.x == x) return kv.b.y;
  if (kv.b.x == INT64_MIN) return dflt;
  const longlong2* t = reinterpret_cast<const longlong2*>(itab + a);
  const uint32_t mask = (1u << m) - 1u;
  uint32_t i = (uint32_t)(((uint64_t)x * 0x9E3779B97F4A7C15ull) >> (64 - m));
  i = (i + 2u) & mask;
  while (true) {
    const longlong2 k = __ldg(t + i);
    if (k.x == x) return k.y;
    if (k.x == INT64_MIN) return dflt;
    i = (i + 1) & mask;
  }
}
// Branch-free MapId from the first two probe slots: *miss = the key is in
// neither and neither is empty (the row probes further on the generic path).
__device__ __forceinline__ int64_t map_sel2(MapProbe2 kv, int64_t x, int64_t dflt, bool* miss) {
  const bool ha = kv.a.x == x, ea = kv.a.x == INT64_MIN, hb = kv.b.x == x, eb = kv.b.x == INT64_MIN;
  const bool xm = x == INT64_MIN;  // never a key (R8 reading: the table's empty marker)
  *miss = !xm && !ha && !ea && !hb && !eb;
  return xm ? dflt : (ha ? kv.a.y : (ea ? dflt : (hb ? kv.b.y : dflt)));
}
__device__ __forceinline__ longlong2 map_first_probe(const int64_t* itab, int64_t a, int m, int64_t x) {
  const longlong2* t = reinterpret_cast<const longlong2*>(itab + a);
  return __ldg(t + (uint32_t)(((uint64_t)x * 0x9E3779B97F4A7C15ull) >> (64 - m)));
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

// Batched forms for N independent elements: every step issues N independent
// loads before any is consumed (memory-level parallelism instead of N
// serial probe chains).
template <int N>
__device__ __forceinline__ void map_lookup_n(const int64_t* itab, int64_t a, int m, int64_t dflt, int64_t (&v)[N],
                                             unsigned act) {  // R8, no INT64_MIN key
  const longlong2* t = reinterpret_cast<const longlong2*>(itab + a);
  const uint32_t mask = (1u << m) - 1u;
  uint32_t idx[N];
  longlong2 kv[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    idx[j] = (uint32_t)(((uint64_t)v[j] * 0x9E3779B97F4A7C15ull) >> (64 - m));
    kv[j] = ((act >> j) & 1u) ? __ldg(t + idx[j]) : make_longlong2(INT64_MIN, 0);
  }
#pragma unroll
  for (int j = 0; j < N; ++j) {
    if (!((act >> j) & 1u)) continue;
    if (v[j] == INT64_MIN) {
      v[j] = dflt;
      continue;
    }
    while (true) {
      if (kv[j].x == v[j]) {
        v[j] = kv[j].y;
        break;
      }
      if (kv[j].x == INT64_MIN) {
        v[j] = dflt;
        break;
      }
      idx[j] = (idx[j] + 1) & mask;
      kv[j] = __ldg(t + idx[j]);
    }
  }
}

// #{i : b[i] <= x} over sorted b[0..m), m >= 1, branchless with a uniform
// step count (R4).
template <int N>
__device__ __forceinline__ void upper_bound_n(const int64_t* b, int m, int64_t (&v)[N], unsigned act) {
  int base[N];
#pragma unroll
  for (int j = 0; j < N; ++j) base[j] = 0;
  int n = m;
  while (n > 1) {
    const int half = n >> 1;
#pragma unroll
    for (int j = 0; j < N; ++j) base[j] += (__ldg(b + base[j] + half) <= v[j]) ? half : 0;
    n -= half;
  }
#pragma unroll
  for (int j = 0; j < N; ++j)
    if ((act >> j) & 1u) v[j] = base[j] + (__ldg(b + base[j]) <= v[j] ? 1 : 0);
}

// Canonical pipeline (rap_internal.h) over N elements: the stages in q.mask,
// in the fixed order Clamp -> MapId -> SigridHash -> Bucketize.  act[j] =
// element j is processed; full[j] = it runs every stage (a valid row) rather
// than q.null_mask (a filled null, R10).  The mask is warp-uniform, so the
// stage tests are uniform branches (one code copy, no per-mask variants:
// instruction-cache footprint matters more than the tests).
template <int N>
__device__ __forceinline__ void canon_apply_nm(const Canon& q, int mask, const int64_t* itab, int64_t (&v)[N],
                                               unsigned act, unsigned full);
template <int N>
__device__ __forceinline__ void canon_apply_n(const Canon& q, const int64_t* itab, int64_t (&v)[N], unsigned act,
                                              unsigned full) {
  canon_apply_nm<N>(q, q.mask, itab, v, act, full);
}
// The stages in `mask` (a subset of q.mask) of the canonical pipeline.
template <int N>
__device__ __forceinline__ void canon_apply_nm(const Canon& q, int mask, const int64_t* itab, int64_t (&v)[N],
                                               unsigned act, unsigned full) {
  // element j runs stage X iff act bit j and (full bit j or X in null_mask).
  // Stage parameters are read once into registers; when every element runs
  // a stage (the steady state: full windows, FillNull first) the stage is
  // straight-line code with no per-element predicate or branch.
  constexpr unsigned kAll = N >= 32 ? 0xffffffffu : ((1u << N) - 1u);
  const int nmask = q.null_mask;
  if (mask & CB_CLAMP) {  // R6
    const int64_t lo = q.lo, hi = q.hi;
    const unsigned on = (nmask & CB_CLAMP) ? act : (act & full);
    if (on == kAll) {
#pragma unroll
      for (int j = 0; j < N; ++j) {
        v[j] = v[j] < lo ? lo : v[j];
        v[j] = v[j] > hi ? hi : v[j];
      }
    } else {
#pragma unroll
      for (int j = 0; j < N; ++j)
        if ((on >> j) & 1u) {
          v[j] = v[j] < lo ? lo : v[j];
          v[j] = v[j] > hi ? hi : v[j];
        }
    }
  }
  if (mask & CB_MAPID)  // R8
    map_lookup_n<N>(itab, q.map_a, q.map_m, q.map_def, v, (nmask & CB_MAPID) ? act : (act & full));
  if (mask & CB_SIGRID) {  // R3
    const unsigned on = (nmask & CB_SIGRID) ? act : (act & full);
    const uint64_t hs = q.hs, M = (uint64_t)q.M;
    if ((M >> 32) == 0) {  // warp-uniform: the 64x32 multiply-high path for the whole batch
      if (on == kAll) {
#pragma unroll
        for (int j = 0; j < N; ++j) {
          const uint64_t h = splitmix_H(hs ^ (uint64_t)v[j]);
          v[j] = (int64_t)(((uint64_t)(uint32_t)(h >> 32) * M + (((uint64_t)(uint32_t)h * M) >> 32)) >> 32);
        }
      } else {
#pragma unroll
        for (int j = 0; j < N; ++j)
          if ((on >> j) & 1u) {
            const uint64_t h = splitmix_H(hs ^ (uint64_t)v[j]);
            v[j] = (int64_t)(((uint64_t)(uint32_t)(h >> 32) * M + (((uint64_t)(uint32_t)h * M) >> 32)) >> 32);
          }
      }
    } else {
#pragma unroll
      for (int j = 0; j < N; ++j)
        if ((on >> j) & 1u) v[j] = (int64_t)__umul64hi(splitmix_H(hs ^ (uint64_t)v[j]), M);
    }
  }
  if (mask & CB_BUCKET)  // R4
    upper_bound_n<N>(itab + q.bk_a, q.bk_m, v, (nmask & CB_BUCKET) ? act : (act & full));
}

// One element through the canonical pipeline (not inlined: cold paths).
static __device__ __noinline__ int64_t canon1(const Canon& q, const int64_t* itab, int64_t x, bool full) {
  int64_t v[1] = {x};
  canon_apply_n<1>(q, itab, v, 1u, full ? 1u : 0u);
  return v[0];
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


// Profiling aid: per-CTA phase stamps (%globaltimer), thread 0 only, enabled
// when the plan allocated a trace buffer (rap_debug_trace).
__device__ __forceinline__ void trace_stamp(const Common& c, int k) {
  if (c.trace != nullptr && threadIdx.x == 0 && (int64_t)blockIdx.x < c.trace_cap) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    c.trace[(int64_t)blockIdx.x * kTracePts + k] = v;
  }
}

// Same, from lane 0 of the calling warp (a warp other than warp 0).
__device__ __forceinline__ void trace_stamp_warp(const Common& c, int k) {
  if (c.trace != nullptr && (threadIdx.x & 31) == 0 && (int64_t)blockIdx.x < c.trace_cap) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    c.trace[(int64_t)blockIdx.x * kTracePts + k] = v;
  }
}

// Profiling aid: clock64 at slot k of this CTA's trace row, once per launch
// (first call wins), after the value `dep` is available.
// Compiled in only with -DRAP_TRACE_CLK (dev builds, scripts/trace.py).
__shared__ unsigned long long s_clk[24];  // trace_clk stamps of this CTA (flushed at kernel end)
__device__ __forceinline__ void trace_clk(const Common& c, int k, long long dep) {
#ifndef RAP_TRACE_CLK
  (void)c;
  (void)k;
  (void)dep;
  if (false)
#endif
  if (c.trace != nullptr && threadIdx.x == 0) {
    asm volatile("" ::"l"(dep));
    if (s_clk[k] == 0) s_clk[k] = clock64();  // shared: no global round trip inside the timed span
  }
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
// Dense block: kDenseBlockRows rows of one column group -> row-major tile via
// smem (a2).  Inputs staged with bulk copies on the CTA mbarrier.
struct CtaState {
  uint64_t bar;
  long long ticket;
  int staged, phase, dgroup;  // dgroup: column group whose DProg is in smem (-1: none)
};

constexpr int kDProgBytes = align_up((int)sizeof(DProg), 16);
static_assert(sizeof(DProg) % 16 == 0, "DProg copies are whole 16-byte words");

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
__device__ __noinline__ void dense_block(const P& p, int gi, int64_t rb, int smem_off, CtaState& cs) {
  // the region is addressed from the dynamic shared array itself (not a
  // pointer argument), so every access compiles to LDS / STS
  unsigned char* smem = rap_dyn_smem + smem_off;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  DProg* dp = reinterpret_cast<DProg*>(smem);
  float* din = reinterpret_cast<float*>(smem + kDProgBytes);  // [16][kDenseBlockRows]
  uint32_t* dbm = reinterpret_cast<uint32_t*>(smem + kDProgBytes + 16 * kDenseBlockRows * 4);  // [16][8]
  float* tile = reinterpret_cast<float*>(smem + kDProgBytes + dense_in_bytes());
  // rows [r0, r0 + nr) of the dense output = raw rows g0 + [0, nr): a
  // sharded plan's dense outputs cover its batch shard only
  const int64_t r0 = rb * kDenseBlockRows;
  const int64_t g0 = p.c.dense_row0 + r0;
  const int nr = (int)min((int64_t)kDenseBlockRows, p.c.n_dense_rows - r0);
  const int nw = (nr + 31) >> 5;
  trace_clk(p.c, 16, 0);
  if (warp == 0) {
    const DProg* g = p.c.dprogs + gi;
    const int nu = __ldg(&g->n_units), no = __ldg(&g->n_ops), nf = __ldg(&g->n_ftab), nc = __ldg(&g->n_cols);
    const int col = lane < nc ? __ldg(&g->cols[lane]) : 0;
    const bool aligned = lane >= nc || ((reinterpret_cast<uintptr_t>(p.dense[col] + g0) & 15) == 0 &&
                                        (p.dvalid[col] == nullptr ||
                                         ((g0 & 31) == 0 &&
                                          (reinterpret_cast<uintptr_t>(p.dvalid[col] + (g0 >> 5)) & 15) == 0)));
    const bool stage = __all_sync(0xffffffffu, aligned) && (nr & 3) == 0 && nc <= 16;
    if (stage) {
      // validity: the 16-byte body by the bulk copy, the <= 3 tail words by
      // plain loads (a bitmap holds exactly ceil(B/32) words: never read past)
      const uint32_t bytes_v = (uint32_t)nr * 4, bytes_b = (uint32_t)(nw * 4) & ~15u;
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
        bulk_g2s(din + lane * kDenseBlockRows, p.dense[col] + g0, bytes_v, &cs.bar);
        if (p.dvalid[col]) {
          if (bytes_b) bulk_g2s(dbm + lane * 8, p.dvalid[col] + (g0 >> 5), bytes_b, &cs.bar);
          for (int i = (int)(bytes_b / 4); i < nw; ++i) dbm[lane * 8 + i] = __ldg(p.dvalid[col] + (g0 >> 5) + i);
        }
      }
    }
    if (lane == 0) cs.staged = stage ? 1 : 0;
  }
  if (cs.dgroup != gi) {
    // the group's program to shared memory once per CTA and group: every
    // thread's loads in flight before any store
    const int4* src = reinterpret_cast<const int4*>(p.c.dprogs + gi);
    int4* dst = reinterpret_cast<int4*>(dp);
    constexpr int kN16 = kDProgBytes / 16, kPer = (kN16 + kThreads - 1) / kThreads;
    int4 r[kPer];
#pragma unroll
    for (int i = 0; i < kPer; ++i)
      if (tid + i * kThreads < kN16) r[i] = __ldg(src + tid + i * kThreads);
#pragma unroll
    for (int i = 0; i < kPer; ++i)
      if (tid + i * kThreads < kN16) dst[tid + i * kThreads] = r[i];
  }
  __syncthreads();
  if (tid == 0) cs.dgroup = gi;
  trace_clk(p.c, 17, 0);
  const int W = dp->width;
  const int LD = W | 1;  // odd row pitch: conflict-free column writes
  if (dp->any_onehot) {
    const int n = nr * LD;  // the tile base is 16-byte aligned
    float4* t4 = reinterpret_cast<float4*>(tile);
    for (int i = tid; i < (n >> 2); i += kThreads) t4[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int i = (n & ~3) + tid; i < n; i += kThreads) tile[i] = 0.0f;
  }
  const bool staged = cs.staged;
  if (staged) mbar_wait(&cs.bar, cs.phase);
  __syncthreads();
  trace_clk(p.c, 18, 0);
  const int nu = dp->n_units;
  // one unit per warp at a time, its rows over the lanes: the unit's
  // descriptor and up to kRegOps dense ops are read once into registers
  // (warp-uniform), then each row is a short straight-line chain
  constexpr int kRegOps = 3;
  for (int u = warp; u < nu; u += kWarps) {
    const DUnit& un = dp->units[u];
    const int kind = un.kind, col = un.col, slot = un.slot, src_col = un.src_col;
    if (kind == U_ONEHOT_G) {  // generic list (R9), program from global memory
      for (int r = lane; r < nr; r += 32) onehot_generic(p, un, g0 + r, tile + r * LD);
      continue;
    }
    const DevOp* uops = un.gops ? p.c.ops : dp->ops;
    const int o0 = un.op_begin, o1 = un.op_end;
    const bool reg_ops = o1 - o0 <= kRegOps;
    int okind[kRegOps];
    float of0[kRegOps], of1[kRegOps];
#pragma unroll
    for (int k = 0; k < kRegOps; ++k) {
      okind[k] = -1;
      of0[k] = of1[k] = 0.0f;
      if (reg_ops && o0 + k < o1) {
        okind[k] = uops[o0 + k].kind;
        of0[k] = uops[o0 + k].f0;
        of1[k] = uops[o0 + k].f1;
      }
    }
    const bool has_bm = p.dvalid[src_col] != nullptr;
    // specialised unit: a staged dense column through [FillNull] [Logit |
    // BoxCox] (the Criteo chains): one uniform dispatch per unit, none per row
    {
      const bool f0 = okind[0] == OK_FILL_F;
      const int t = f0 ? okind[1] : okind[0];
      const int rest = f0 ? okind[2] : okind[1];
      const int tp = f0 ? 1 : 0;
      if (staged && kind == U_DENSE && reg_ops && rest < 0 && (t < 0 || t == OK_LOGIT || t == OK_BOXCOX)) {
        const float fill = of0[0], a = of0[tp], b = of1[tp];
        const float* xin = din + slot * kDenseBlockRows;
        const uint32_t* bmp = dbm + slot * 8;
        float* tc = tile + col;
        auto in = [&](int r) -> float {  // R14 null -> NaN, then R10
          const uint32_t w = has_bm ? bmp[r >> 5] : 0xffffffffu;
          float x = ((w >> (r & 31)) & 1u) ? xin[r] : __int_as_float(0x7fc00000);
          if (f0 && isnan(x)) x = fill;
          return x;
        };
        if (t == OK_LOGIT) {  // R11
          for (int r = lane; r < nr; r += 32) {
            const float x = in(r);
            const float z = x < a ? a : (x > b ? b : x);
            tc[r * LD] = logf(__fdiv_rn(z, __fsub_rn(1.0f, z)));
          }
        } else if (t == OK_BOXCOX && a == 0.0f) {  // R12, lambda = 0
          for (int r = lane; r < nr; r += 32) tc[r * LD] = logf(in(r));
        } else if (t == OK_BOXCOX) {  // R12
          for (int r = lane; r < nr; r += 32) tc[r * LD] = __fdiv_rn(expm1f(__fmul_rn(a, logf(in(r)))), a);
        } else {
          for (int r = lane; r < nr; r += 32) tc[r * LD] = in(r);
        }
        continue;
      }
    }
    const float* uft = un.gops ? p.c.ftab : dp->ftab;
    for (int r = lane; r < nr; r += 32) {
      float x;
      if (staged) {
        const uint32_t w = has_bm ? dbm[slot * 8 + (r >> 5)] : 0xffffffffu;
        x = ((w >> (r & 31)) & 1u) ? din[slot * kDenseBlockRows + r] : __int_as_float(0x7fc00000);
      } else {
        x = dense_raw(p, src_col, g0 + r);
      }
      if (reg_ops) {
#pragma unroll
        for (int k = 0; k < kRegOps; ++k) {  // R10-R12, same expressions as apply_dense_ops
          const int ok = okind[k];
          if (ok == OK_FILL_F) {
            if (isnan(x)) x = of0[k];
          } else if (ok == OK_LOGIT) {
            const float z = x < of0[k] ? of0[k] : (x > of1[k] ? of1[k] : x);
            x = logf(__fdiv_rn(z, __fsub_rn(1.0f, z)));
          } else if (ok == OK_BOXCOX) {
            const float lam = of0[k];
            if (lam == 0.0f) {
              x = logf(x);
            } else {
              const float v = __fmul_rn(lam, logf(x));
              x = __fdiv_rn(expm1f(v), lam);
            }
          }
        }
      } else {
        x = apply_dense_ops(uops, x, o0, o1);
      }
      if (kind == U_DENSE) {
        tile[r * LD + col] = x;
      } else if (un.xcap > 0) {  // U_ONEHOT_DB
        const int64_t bidx = un.gops ? upper_bound(uft + un.btab, un.bm, x) : upper_bound_s(uft + un.btab, un.bm, x);
        const int64_t id = apply_id_ops(uops, p.c.itab, 0, bidx, un.iop_begin, un.iop_end);
        const int64_t d = id - un.k0;
        if (d >= 0 && d < un.width) tile[r * LD + col + (int)d] = 1.0f;
      }
    }
  }
  __syncthreads();
  trace_clk(p.c, 19, 0);
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
  trace_clk(p.c, 20, 0);
  if (tid == 0 && staged) cs.phase ^= 1;
}

}  // namespace rapk
