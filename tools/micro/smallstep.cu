#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
constexpr unsigned FULL = 0xffffffffu;
constexpr unsigned long long kS = ~0ull;
__device__ __forceinline__ unsigned long long ldv(unsigned a){unsigned long long v; asm volatile("ld.volatile.shared.u64 %0, [%1];":"=l"(v):"r"(a):"memory"); return v;}
__device__ __forceinline__ void stv(unsigned a, unsigned long long v){asm volatile("st.volatile.shared.u64 [%0], %1;"::"r"(a),"l"(v):"memory");}
// chain: row i deps on i-1 (entries: [i-1, i]) ; variant 0: loop as in k_solve_small; 1: no inner while
// minimal in-warp smem ping: row i waits for x[i-1] and stores x[i] (V 2: vote loop, 3: + fp64 step)
template <int V>
__global__ void kp(int n, long long *out, double *xo) {
  extern __shared__ __align__(16) unsigned char sm[];
  unsigned long long *xs = (unsigned long long*)sm;
  const int T = blockDim.x, tid = threadIdx.x;
  for (int k = tid; k < n; k += T) xs[k] = kS;
  __syncthreads();
  const unsigned xs_s = (unsigned)__cvta_generic_to_shared(xs);
  long long t0 = clock64();
  int r = tid; bool act = r < n;
  while (__any_sync(FULL, act)) {
    if (act) {
      unsigned long long v = r == 0 ? 0ull : ldv(xs_s + 8u*(unsigned)(r-1));
      if (v != kS) {
        double a = __longlong_as_double(v);
        if (V == 3) a = __dadd_rn(1.0, __dmul_rn(a, -0.5));
        stv(xs_s + 8u*(unsigned)r, V == 3 ? __double_as_longlong(a) : v + 1);
        r += T; act = r < n;
      }
    }
  }
  long long t1 = clock64();
  __syncthreads();
  if (tid == T - 1) out[0] = t1 - t0;
  for (int k = tid; k < n; k += T) xo[k] = __longlong_as_double(xs[k]);
}
// V 4: branch-free pass (predicated poll and store), V 5: V 4 + a second poll in the same pass
template <int V>
__global__ void kq(int n, long long *out, double *xo) {
  extern __shared__ __align__(16) unsigned char sm[];
  unsigned long long *xs = (unsigned long long*)sm;
  const int T = blockDim.x, tid = threadIdx.x;
  for (int k = tid; k < n; k += T) xs[k] = kS;
  __syncthreads();
  const unsigned xs_s = (unsigned)__cvta_generic_to_shared(xs);
  long long t0 = clock64();
  int r = tid; bool act = r < n;
  unsigned long long v = 0;
  while (__any_sync(FULL, act)) {
    const unsigned pa = xs_s + 8u*(unsigned)(r > 0 ? r - 1 : 0);
    v = r == 0 ? 0ull : ldv(pa);
    bool rdy = act && v != kS;
    if (V == 5 && !rdy && act) { v = ldv(pa); rdy = v != kS; }
    const unsigned long long w = v + 1;
    asm volatile("{.reg .pred p; setp.ne.u32 p, %2, 0; @p st.volatile.shared.u64 [%0], %1;}"
                 :: "r"(xs_s + 8u*(unsigned)(r < n ? r : 0)), "l"(w), "r"((unsigned)rdy) : "memory");
    r += rdy ? T : 0; act = r < n;
  }
  long long t1 = clock64();
  __syncthreads();
  if (tid == T - 1) out[0] = t1 - t0;
  for (int k = tid; k < n; k += T) xo[k] = __longlong_as_double(xs[k]);
}
template <int V>
__global__ void k(int n, long long *out, double *xo) {
  extern __shared__ __align__(16) unsigned char sm[];
  unsigned long long *xs = (unsigned long long*)sm;
  int *cs = (int*)(xs + n);
  double *vs = (double*)(cs + 2*n);
  const int T = blockDim.x, tid = threadIdx.x;
  for (int k = tid; k < n; k += T) { xs[k] = kS; cs[2*k] = k-1; cs[2*k+1] = k; vs[2*k] = -0.5; vs[2*k+1] = 1.0; }
  __syncthreads();
  const unsigned xs_s = (unsigned)__cvta_generic_to_shared(xs);
  long long t0 = clock64();
  int r = tid, j = 0, e = 0, i = 0; double ls = 0;
  auto load = [&]() { i = r; j = (i == 0) ? 1 : 2*i; e = 2*i+1; ls = 0; };
  bool act = r < n; if (act) load();
  while (__any_sync(FULL, act)) {
    if (!act) continue;
    if (V == 0) {
      while (j != e) {
        unsigned long long v = ldv(xs_s + 8u*(unsigned)cs[j]);
        if (v == kS) break;
        ls = __dadd_rn(ls, __dmul_rn(vs[j], __longlong_as_double(v)));
        j++;
      }
      if (j != e) continue;
    } else {
      if (j != e) {
        unsigned long long v = ldv(xs_s + 8u*(unsigned)cs[j]);
        if (v == kS) continue;
        ls = __dadd_rn(ls, __dmul_rn(vs[j], __longlong_as_double(v)));
        j++;
        if (j != e) continue;
      }
    }
    double a = __dsub_rn(1.0, ls);
    stv(xs_s + 8u*(unsigned)i, __double_as_longlong(a));
    r += T; act = r < n; if (act) load();
  }
  long long t1 = clock64();
  __syncthreads();
  if (tid == T - 1) out[0] = t1 - t0;
  for (int k = tid; k < n; k += T) xo[k] = __longlong_as_double(xs[k]);
}
int main() {
  int n = 1024; long long *o; double *x; cudaMalloc(&o, 8); cudaMalloc(&x, 8*n);
  size_t sm = n*8 + n*8 + n*16;
  for (int T : {32, 64, 1024}) {
    for (int v = 0; v < 2; ++v) {
      for (int rep = 0; rep < 3; ++rep) {
        if (v == 0) k<0><<<1, T, sm>>>(n, o, x); else k<1><<<1, T, sm>>>(n, o, x);
      }
      long long h; cudaMemcpy(&h, o, 8, cudaMemcpyDeviceToHost);
      double xl; cudaMemcpy(&xl, x + n - 1, 8, cudaMemcpyDeviceToHost);
      printf("T=%d variant %d: %.1f cycles per hop (x_last %g) %s\n", T, v, (double)h / n, xl, cudaGetErrorString(cudaGetLastError()));
    }
    for (int v = 4; v < 6; ++v) {
      for (int rep = 0; rep < 3; ++rep) {
        if (v == 4) kq<4><<<1, T, sm>>>(n, o, x); else kq<5><<<1, T, sm>>>(n, o, x);
      }
      long long h; cudaMemcpy(&h, o, 8, cudaMemcpyDeviceToHost);
      printf("T=%d branch-free variant %d: %.1f cycles per hop %s\n", T, v, (double)h / n, cudaGetErrorString(cudaGetLastError()));
    }
    for (int v = 2; v < 4; ++v) {
      for (int rep = 0; rep < 3; ++rep) {
        if (v == 2) kp<2><<<1, T, sm>>>(n, o, x); else kp<3><<<1, T, sm>>>(n, o, x);
      }
      long long h; cudaMemcpy(&h, o, 8, cudaMemcpyDeviceToHost);
      printf("T=%d ping variant %d: %.1f cycles per hop %s\n", T, v, (double)h / n, cudaGetErrorString(cudaGetLastError()));
    }
  }
}
