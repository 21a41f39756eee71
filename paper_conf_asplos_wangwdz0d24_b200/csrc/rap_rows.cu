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
#include <string.h>

#ifndef RAP_ROWS_PLAIN_STORES
#define RAP_ST_CS 1  // streaming output stores (rap_rows_skel.cuh)
#endif
#include "rap_rows_interp.cuh"

namespace rapk {

#ifndef RAP_RB_MIN_CTAS
#define RAP_RB_MIN_CTAS 2
#endif
template <int MD, int MS, bool kSmall>
__global__ void __launch_bounds__(kRbChunk, RAP_RB_MIN_CTAS) rap_rows_kernel(const __grid_constant__ RbParams<MD, MS> p) {
  rows_body<InterpPolicy, MD, MS, kSmall>(p);
}

template <int MD, int MS, bool kSmall>
static int launch_rows_t(const Common& c, const RbGeom& g, const LaunchRaw& raw, int smem, cudaStream_t st) {
  static_assert(sizeof(RbParams<MD, MS>) <= 32000, "kernel parameter block too large");
  const int rc = ensure_dyn_smem(reinterpret_cast<const void*>(rap_rows_kernel<MD, MS, kSmall>), smem);
  if (rc != 0) return rc;
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
  cfg.gridDim = dim3((unsigned)(g.n_rb * g.n_fg + g.n_dcta));
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

int rows_smem_bytes(int dense_bytes, int max_fl, int max_cols, int n_memo, int n_sparse_out, int len_cache,
                    int id_slots, int pitch, int feat_recs, int tab_bytes) {
  int o = rb_region0(dense_bytes, n_memo, n_sparse_out);
  o += 2 * rb_align(max_fl * 8 * 8);
  o += rb_align(max_fl * 8);
  if (feat_recs) o += rb_align(max_fl * (int)sizeof(RbF));
  o += rb_align(max_cols * (pitch > 0 ? pitch : kRbPitch) * 4);
  o += rb_align(max_cols * 8 * 4);
  if (len_cache) o += rb_align(max_fl * kRbChunk * 2);
  if (id_slots > 0) o += rb_align(id_slots * 8) + id_slots * kRbIdCap * 8;
  if (tab_bytes > 0) o = rb_align(o) + tab_bytes;
  return o;
}

int rows_occupancy(int smem_bytes, int* ctas_per_sm) {
  const void* k32 = reinterpret_cast<const void*>(rap_rows_kernel<kRbMaxDense, kRbMaxCols, true>);
  const void* k64 = reinterpret_cast<const void*>(rap_rows_kernel<kRbMaxDense, kRbMaxCols, false>);
  int rc = ensure_dyn_smem(k32, smem_bytes);
  if (rc == 0) rc = ensure_dyn_smem(k64, smem_bytes);
  if (rc != 0) return rc;
  return (int)cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, k32, kRbChunk, smem_bytes);
}

}  // namespace rapk
