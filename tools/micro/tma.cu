// Throughput of 1-D TMA bulk copies (cp.async.bulk global->shared, mbarrier complete_tx)
// of a given size: every CTA (one thread issues) streams `iters` copies through a ring of S slots.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "../../paper_conf_icpp_suz0hw0w20_b200/csrc/ptx.cuh"
using namespace sptrsv_dev;
__global__ void k(const char* src, long long span, int bytes, int iters, int S, unsigned long long* sink) {
  extern __shared__ __align__(16) unsigned char sm[];
  __shared__ __align__(8) unsigned long long bars[16];
  if (threadIdx.x != 0) return;
  for (int s = 0; s < S; ++s) mbar_init(smem_u32(&bars[s]), 1);
  fence_mbar_init();
  uint64_t pol = policy_evict_first();
  unsigned long long acc = 0;
  long long off = (long long)blockIdx.x * bytes * iters % span;
  for (int it = 0; it < iters; ++it) {
    int s = it % S;
    if (it >= S) { unsigned par = ((it / S) - 1) & 1; while (!mbar_try_wait(smem_u32(&bars[s]), par)) {} acc += sm[s * bytes]; }
    mbar_arrive_expect_tx(smem_u32(&bars[s]), bytes);
    bulk_g2s(smem_u32(sm + s * bytes), src + (off & ~15ll), bytes, smem_u32(&bars[s]), pol);
    off = (off + bytes) % (span - bytes);
  }
  for (int it = iters; it < iters + S; ++it) { int s = it % S; unsigned par = ((it / S) - 1) & 1; while (!mbar_try_wait(smem_u32(&bars[s]), par)) {} }
  sink[blockIdx.x] = acc;
}
int main() {
  long long span = 512ll << 20; char* src; cudaMalloc(&src, span); cudaMemset(src, 1, span);
  unsigned long long* sink; cudaMalloc(&sink, 8 * 4096);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int bytes : {512, 1024, 4096, 16384}) for (int S : {2, 4, 8}) for (int ctas : {148, 592}) {
    int iters = (int)((256ll << 20) / ((long long)bytes * ctas)); if (iters < 8) iters = 8;
    size_t smem = (size_t)bytes * S; if (smem > 200 * 1024) continue;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    k<<<ctas, 32, smem>>>(src, span, bytes, iters, S, sink); cudaDeviceSynchronize();
    cudaEventRecord(a); k<<<ctas, 32, smem>>>(src, span, bytes, iters, S, sink); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    double tot = (double)bytes * iters * ctas;
    printf("bytes=%6d S=%d ctas=%4d : %.2f TB/s  %.1f copies/us/SM\n", bytes, S, ctas, tot / (ms * 1e-3) / 1e12,
           (double)iters * ctas / (ms * 1e3) / 148.0);
  }
  return 0;
}
