// Micro-benchmark: cost of one "local round" of an in-warp dependency chain.
// One warp; lane l waits for lane l-1's value in smem, then computes and publishes.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define FULL 0xffffffffu
__device__ __forceinline__ unsigned long long lds(unsigned a){unsigned long long v; asm volatile("ld.volatile.shared.u64 %0,[%1];":"=l"(v):"r"(a):"memory"); return v;}
__device__ __forceinline__ void sts(unsigned a, unsigned long long v){asm volatile("st.volatile.shared.u64 [%0],%1;"::"r"(a),"l"(v):"memory");}

template<int V>
__global__ void k(double* out, unsigned long long* rec, double* x, long long* cyc, int reps){
  __shared__ unsigned long long xc[64];
  int lane = threadIdx.x;
  unsigned base = (unsigned)__cvta_generic_to_shared(xc);
  double d = 2.0, b = 1.0, nv = -1.0, s = 0;
  long long t0 = 0, tot = 0;
  for (int r = 0; r < reps; ++r) {
    xc[lane] = ~0ull; xc[32+lane] = ~0ull;
    __syncwarp();
    t0 = __shfl_sync(FULL, (long long)clock64(), 0);
    bool done = false; s = 0;
    int nc = lane - 1;
    if (lane == 0) { double xi = b / d; sts(base + 8*lane, __double_as_longlong(xi)); done = true; }
    while (true) {
      bool lp = false;
      if (!done) {
        unsigned long long v = lds(base + 8*nc);
        if (v != ~0ull) {
          s = s + nv * __longlong_as_double(v);
          double xi;
          if (V >= 1) xi = __ddiv_rn(b - s, d); else xi = (b - s) * 0.5;
          unsigned long long bits = __double_as_longlong(xi);
          sts(base + 8*lane, bits);
          if (V >= 2) {  // global stores like publish
            asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(rec + 2*(r*32+lane)), "l"(bits), "l"(bits) : "memory");
            x[r*32+lane] = xi;
          }
          done = true; lp = true;
        }
      }
      if (V >= 3) { if (!__ballot_sync(FULL, !done)) break; if (!__ballot_sync(FULL, lp)) continue; }
      else { if (!__ballot_sync(FULL, !done)) break; }
    }
    if (lane == 31) { tot += clock64() - t0; }

  }
  if (lane == 31) { cyc[0] = tot; out[0] = s; }
}

template<int V> void run(const char* name, int blocks) {
  double* out; unsigned long long* rec; double* x; long long* cyc;
  int reps = 1000;
  cudaMalloc(&out, 8); cudaMalloc(&rec, 16*32*reps); cudaMalloc(&x, 8*32*reps); cudaMalloc(&cyc, 8);
  k<V><<<blocks, 32>>>(out, rec, x, cyc, reps); cudaDeviceSynchronize();
  k<V><<<blocks, 32>>>(out, rec, x, cyc, reps);
  long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  printf("%-40s blocks=%4d  cycles/round = %.1f\n", name, blocks, (double)c / reps / 31.0);
  cudaFree(out); cudaFree(rec); cudaFree(x); cudaFree(cyc);
}
int main(){
  run<0>("lds+dmul+dadd+sts (no div)", 1);
  run<1>("+ ddiv", 1);
  run<2>("+ global publish stores", 1);
  run<3>("+ progress ballot", 1);
  run<2>("+ global publish stores", 148*16);
  return 0;
}
