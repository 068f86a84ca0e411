// Same-address atomicAdd throughput: every warp's lane 0 takes `per` tickets in a loop.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(unsigned* ctr, int per, unsigned* sink) {
  if (threadIdx.x & 31) return;
  unsigned acc = 0;
  for (int i = 0; i < per; ++i) acc += atomicAdd(ctr, 1u);
  if (acc == 7) sink[0] = acc;
}
int main() {
  unsigned *ctr, *sink; cudaMalloc(&ctr, 4); cudaMalloc(&sink, 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  int grids[] = {148, 592, 1184, 2368};
  for (int g : grids) {
    cudaMemset(ctr, 0, 4);
    k<<<g, 256>>>(ctr, 16, sink); cudaDeviceSynchronize();
    cudaEventRecord(a); k<<<g, 256>>>(ctr, 16, sink); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    double n = (double)g * 8 * 16;
    printf("warps=%6d atomics=%8.0f  %.3f ms  -> %.2f atomics/ns\n", g * 8, n, ms, n / (ms * 1e6));
  }
  return 0;
}
