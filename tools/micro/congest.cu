// Flag-hop latency under polling load: 2 threads ping-pong (FUSED-style value
// polls) while `nbg` background warps poll random never-ready 16-byte records
// with a given nanosleep between polls.  Prints ns per one-way hop.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ void ldv2(const unsigned long long* p, unsigned long long& a, unsigned long long& b){
  asm volatile("ld.relaxed.gpu.global.v2.u64 {%0,%1},[%2];":"=l"(a),"=l"(b):"l"(p):"memory");}
__device__ __forceinline__ void stv2(unsigned long long* p, unsigned long long a, unsigned long long b){
  asm volatile("st.relaxed.gpu.global.v2.u64 [%0],{%1,%2};"::"l"(p),"l"(a),"l"(b):"memory");}
__device__ volatile int stop_flag;
__global__ void k(unsigned long long* rec, unsigned long long* pp, int iters, int sleep_ns, long long nrec,
                  unsigned long long* out, unsigned long long* sink) {
  if (blockIdx.x < 2) {
    if (threadIdx.x) return;
    int me = blockIdx.x;
    unsigned long long* my = pp + 16*me; unsigned long long* ot = pp + 16*(1-me);
    unsigned long long t0 = 0;
    asm volatile("mov.u64 %0, %%globaltimer;":"=l"(t0));
    for (int it = 1; it <= iters; ++it) {
      for (int ph = 0; ph < 2; ++ph) {
        bool send = (ph == 0) == (me == 0);
        if (send) stv2(my, it, it);
        else { unsigned long long a, b; do { ldv2(ot, a, b); } while (a != (unsigned long long)it); }
      }
    }
    unsigned long long t1; asm volatile("mov.u64 %0, %%globaltimer;":"=l"(t1));
    if (me == 0) { out[0] = t1 - t0; stop_flag = 1; }
    return;
  }
  // background pollers
  unsigned long long acc = 0, x = (blockIdx.x * 1315423911ull + threadIdx.x * 2654435761ull) | 1;
  while (!stop_flag) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    unsigned long long a, b; ldv2(rec + 2 * (x % nrec), a, b); acc += a ^ b;
    if (sleep_ns) __nanosleep(sleep_ns);
  }
  if (acc == 12345) sink[0] = acc;
}
int main() {
  long long nrec = 1 << 21;  // 32 MB of records
  unsigned long long *rec, *pp, *out, *sink;
  cudaMalloc(&rec, 16 * nrec); cudaMemset(rec, 0, 16 * nrec);
  cudaMalloc(&pp, 512); cudaMalloc(&out, 8); cudaMalloc(&sink, 8);
  int nsms; cudaDeviceGetAttribute(&nsms, cudaDevAttrMultiProcessorCount, 0);
  int bgs[] = {0, 148, 592, 1184, 2368, 4736};
  int sleeps[] = {0, 256, 1024};
  for (int si = 0; si < 3; ++si) for (int bi = 0; bi < 6; ++bi) {
    int zero = 0; cudaMemcpyToSymbol(stop_flag, &zero, 4); cudaMemset(pp, 0, 512);
    int blocks = 2 + bgs[bi] / 8;  // 8 warps per background block
    k<<<blocks, 256>>>(rec, pp, 20000, sleeps[si], nrec, out, sink);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long t; cudaMemcpy(&t, out, 8, cudaMemcpyDeviceToHost);
    printf("bg_warps=%5d sleep=%4dns  hop=%.1f ns %s\n", (blocks - 2) * 8, sleeps[si], t / 40000.0, e ? cudaGetErrorString(e) : "");
  }
  return 0;
}
