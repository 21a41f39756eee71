// Microbenchmark (dev tool): fixed cost of the launch shapes the fused kernel
// can use on B200 -- plain vs cooperative launch, a large __grid_constant__
// parameter block, and a grid-wide "all CTAs published" wait over epoch-tagged
// words (the scan's dependency).  Per-launch times from CUDA events over
// back-to-back launches, and inside a CUDA graph.
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>

struct Big { unsigned long long w[1024]; };  // 8 KB parameter block

__global__ void k_empty(int* o) { if (threadIdx.x == 9999) o[0] = 1; }
__global__ void k_big(const __grid_constant__ Big b, int* o) {
  if (threadIdx.x == 0 && b.w[blockIdx.x & 1023] == 12345) o[0] = 1;
}
// every CTA publishes an epoch-tagged word, then warp 0 waits until all G words carry the epoch
__global__ void k_wait(unsigned long long* agg, unsigned long long* epoch_p, int* o) {
  const unsigned long long ep = *(volatile unsigned long long*)epoch_p;
  const unsigned long long tag = ep + 1;
  if (threadIdx.x == 0) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(agg + blockIdx.x), "l"(tag << 44) : "memory");
  }
  if (threadIdx.x < 32) {
    for (int j0 = 0; j0 < (int)gridDim.x; j0 += 32) {
      const int j = j0 + threadIdx.x;
      bool ok = false;
      while (!ok) {
        unsigned long long v = (1ull << 63);
        if (j < (int)gridDim.x) asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(agg + j) : "memory");
        ok = j >= (int)gridDim.x || (v >> 44) == tag;
        ok = __all_sync(0xffffffffu, ok);
      }
    }
  }
  __syncthreads();
  // last CTA out advances the epoch
  __shared__ int last;
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd((unsigned long long*)(epoch_p + 1), 1ull) == gridDim.x - 1;
  }
  __syncthreads();
  if (last && threadIdx.x == 0) {
    epoch_p[1] = 0;
    __threadfence();
    *(volatile unsigned long long*)epoch_p = ep + 1;
  }
}

static cudaError_t launch(int kind, int grid, bool coop, cudaStream_t st, int* o, unsigned long long* agg,
                          unsigned long long* ep, const Big& big) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(256);
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = coop ? 1 : 0;
  if (kind == 0) return cudaLaunchKernelEx(&cfg, k_empty, o);
  if (kind == 1) return cudaLaunchKernelEx(&cfg, k_big, big, o);
  return cudaLaunchKernelEx(&cfg, k_wait, agg, ep, o);
}

int main() {
  int* o;
  unsigned long long *agg, *ep;
  cudaMalloc(&o, 64);
  cudaMalloc(&agg, 8 * 4096);
  cudaMemset(agg, 0, 8 * 4096);
  cudaMalloc(&ep, 64);
  cudaMemset(ep, 0, 64);
  Big big;
  memset(&big, 0, sizeof(big));
  cudaStream_t st;
  cudaStreamCreate(&st);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const char* names[3] = {"empty", "param8KB", "gridwait"};
  const int N = 2000;
  for (int kind = 0; kind < 3; ++kind)
    for (int grid : {148, 296, 444, 592})
      for (int coop = 0; coop < 2; ++coop) {
        for (int i = 0; i < 20; ++i) launch(kind, grid, coop, st, o, agg, ep, big);
        cudaEventRecord(a, st);
        for (int i = 0; i < N; ++i) launch(kind, grid, coop, st, o, agg, ep, big);
        cudaEventRecord(b, st);
        cudaEventSynchronize(b);
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        // graph
        cudaGraph_t g;
        cudaGraphExec_t ge;
        cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
        for (int i = 0; i < 100; ++i) launch(kind, grid, coop, st, o, agg, ep, big);
        cudaStreamEndCapture(st, &g);
        float gms = -1;
        if (cudaGraphInstantiate(&ge, g, 0) == cudaSuccess) {
          cudaGraphLaunch(ge, st);
          cudaStreamSynchronize(st);
          cudaEventRecord(a, st);
          for (int r = 0; r < 20; ++r) cudaGraphLaunch(ge, st);
          cudaEventRecord(b, st);
          cudaEventSynchronize(b);
          cudaEventElapsedTime(&gms, a, b);
          gms /= 20 * 100;
          cudaGraphExecDestroy(ge);
        }
        cudaGraphDestroy(g);
        printf("%-9s grid %4d %-5s stream %6.2f us/launch   graph %6.2f us/launch   %s\n", names[kind], grid,
               coop ? "coop" : "plain", ms * 1e3 / N, gms * 1e3, cudaGetErrorString(cudaGetLastError()));
      }
  return 0;
}
