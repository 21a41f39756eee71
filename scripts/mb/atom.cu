// Microbenchmark (dev tool): cost of a per-CTA ticket atomic in the prologue.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k0(unsigned long long* s, long long* o) {  // no atomic
  __shared__ int r; if (threadIdx.x == 0) r = blockIdx.x; __syncthreads(); if (r == -1) o[0] = 1; }
__global__ void k1(unsigned long long* s, long long* o) {  // ticket + done atomics, same line
  __shared__ unsigned long long r; if (threadIdx.x == 0) r = atomicAdd(s + 2, 1ull); __syncthreads();
  if (threadIdx.x == 0) { unsigned long long d = atomicAdd(s, 1ull); if (d == gridDim.x - 1) { s[0] = 0; s[2] = 0; } }
  if (r == 0xffffffffull) o[0] = 1; }
__global__ void k2(unsigned long long* s, long long* o) {  // ticket only
  __shared__ unsigned long long r; if (threadIdx.x == 0) r = atomicAdd(s + 2, 1ull); __syncthreads();
  if (r == 0xffffffffull) o[0] = 1; }
int main() {
  unsigned long long* s; long long* o; cudaMalloc(&s, 4096); cudaMemset(s, 0, 4096); cudaMalloc(&o, 64);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b); float ms;
  for (int g : {148, 592, 1184}) {
    for (int v = 0; v < 3; ++v) {
      for (int w = 0; w < 10; ++w) { if (v == 0) k0<<<g, 256>>>(s, o); else if (v == 1) k1<<<g, 256>>>(s, o); else k2<<<g, 256>>>(s, o); }
      cudaEventRecord(a);
      for (int i = 0; i < 200; ++i) { if (v == 0) k0<<<g, 256>>>(s, o); else if (v == 1) k1<<<g, 256>>>(s, o); else k2<<<g, 256>>>(s, o); }
      cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
      printf("grid %4d variant %d: %.2f us/launch\n", g, v, ms * 1e3 / 200);
    }
  }
  // graph of 200 launches of k0
  cudaStream_t st; cudaStreamCreate(&st); cudaGraph_t gr; cudaGraphExec_t ge;
  cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < 200; ++i) k0<<<592, 256, 0, st>>>(s, o);
  cudaStreamEndCapture(st, &gr); cudaGraphInstantiate(&ge, gr, 0); cudaGraphLaunch(ge, st); cudaStreamSynchronize(st);
  cudaEventRecord(a, st); cudaGraphLaunch(ge, st); cudaEventRecord(b, st); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
  printf("graph of 200 x k0 592: %.2f us/launch\n", ms * 1e3 / 200);
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
