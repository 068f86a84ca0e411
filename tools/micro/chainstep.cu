// Latency of one step of the in-warp chain (ENGINE_CHAIN): dependent fp64 op latencies,
// the 64-bit shuffle, and the whole step (shfl -> mul/add -> sub -> division -> shfl) with
// the verified division vs plain __ddiv_rn vs an unchecked Markstein step.  One warp, clock64.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

struct Diag {
    double d, r;
    __device__ __forceinline__ void init(double dv) {
        d = dv;
        const double ad = fabs(dv);
        r = (ad >= 0x1p-400 && ad <= 0x1p400) ? __drcp_rn(dv) : 0.0;
    }
    __device__ __forceinline__ double div(double a) const {
        const double q0 = __dmul_rn(a, r);
        const double e = __fma_rn(-q0, d, a);
        const double q = __fma_rn(e, r, q0);
        const double e2 = __fma_rn(-q, d, a);
        const unsigned long long qb = (unsigned long long)__double_as_longlong(q);
        const unsigned long long ex = qb & 0x7FF0000000000000ull;
        const unsigned long long sh = (qb & 0x000FFFFFFFFFFFFFull) ? (53ull << 52) : (54ull << 52);
        const double thr = fabs(d) * __longlong_as_double((long long)(ex - sh));
        const double aa = fabs(a);
        if (r != 0.0 && aa >= 0x1p-400 && aa <= 0x1p400 && fabs(e2) < thr) return q;
        return __ddiv_rn(a, d);
    }
    __device__ __forceinline__ double div_fast(double a) const {  // unchecked candidate
        const double q0 = __dmul_rn(a, r);
        const double e = __fma_rn(-q0, d, a);
        return __fma_rn(e, r, q0);
    }
    // verified, slow path out of line (never if-converted)
    __device__ __forceinline__ double div_branch(double a) const {
        const double q0 = __dmul_rn(a, r);
        const double e = __fma_rn(-q0, d, a);
        const double q = __fma_rn(e, r, q0);
        const double e2 = __fma_rn(-q, d, a);
        const unsigned long long qb = (unsigned long long)__double_as_longlong(q);
        const unsigned long long ex = qb & 0x7FF0000000000000ull;
        const unsigned long long sh = (qb & 0x000FFFFFFFFFFFFFull) ? (53ull << 52) : (54ull << 52);
        const double thr = fabs(d) * __longlong_as_double((long long)(ex - sh));
        const double aa = fabs(a);
        if (__builtin_expect(r != 0.0 && aa >= 0x1p-400 && aa <= 0x1p400 && fabs(e2) < thr, 1)) return q;
        double out;
        asm volatile("{ .reg .pred p; setp.ne.s32 p, 1, 0; @p div.rn.f64 %0, %1, %2; }" : "=d"(out) : "d"(a), "d"(d));
        return out;
    }
};

template <int V>
__global__ void k_chain(double *out, long long *cyc, int steps, double d0, double v0, double b0,
                        unsigned long long *rec = nullptr, double *xg = nullptr) {
    __shared__ double s_x[64];
    const int lane = threadIdx.x;
    Diag dg;
    dg.init(d0 + lane * 1e-3);
    const double nv = v0, bk = b0;
    double ls = 0.0, x = 1.0;
    long long t0 = clock64();
    for (int s = 0; s < steps; ++s) {
        const int owner = s & 31;
        double xo = 0.0;
        if (lane == owner) {
            const double a = __dsub_rn(bk, ls);
            if (V == 0) xo = dg.div(a);
            if (V == 1) xo = __ddiv_rn(a, dg.d);
            if (V == 2) xo = dg.div_fast(a);
            if (V == 3) xo = dg.div_branch(a);
            if (V == 4) xo = a;  // no division
            if (V >= 5) xo = dg.div_fast(a);
        }
        x = __shfl_sync(0xffffffffu, xo, owner);
        if (V >= 5 && lane == owner) {
            unsigned long long bits = __double_as_longlong(x), e = 1ull << 32;
            s_x[s & 63] = x;
            if (V >= 6) {
                asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(rec + 2 * (size_t)(s & 4095)),
                             "l"(e | (bits & 0xffffffffull)), "l"(e | (bits >> 32)) : "memory");
                xg[s & 4095] = x;
            }
            if (V >= 7) {
                unsigned long long t;
                asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
                xg[4096 + (s & 4095)] = (double)t;
            }
        }
        if (lane == ((s + 1) & 31)) ls = __dadd_rn(0.0, __dmul_rn(nv, x));
    }
    long long t1 = clock64();
    if (lane == 0) {
        out[0] = x + ls;
        cyc[V] = (t1 - t0) / steps;
    }
}

// The kernel's step (solve_chain.cuh section C) with parts switched off: W bit0 = exactness
// check + vote, bit1 = per-step record store, bit2 = consume via nc compare / advance.
__device__ __forceinline__ bool exact_chk(const Diag &g, double a, double q) {
    const double e2 = __fma_rn(-q, g.d, a);
    const unsigned long long qb = (unsigned long long)__double_as_longlong(q);
    const unsigned long long ex = qb & 0x7FF0000000000000ull;
    const unsigned long long sh = (qb & 0x000FFFFFFFFFFFFFull) ? (53ull << 52) : (54ull << 52);
    const double thr = fabs(g.d) * __longlong_as_double((long long)(ex - sh));
    const double aa = fabs(a);
    return g.r != 0.0 && aa >= 0x1p-400 && aa <= 0x1p400 && fabs(e2) < thr;
}
template <int W>
__global__ void k_step(long long *cyc, int steps, double d0, unsigned long long *rec, int *cols) {
    const int lane = threadIdx.x;
    Diag dg;
    dg.init(d0 + lane * 1e-3);
    double ls = 0.0, bk = 1.0, nv = -1.0, xm = 0;
    int nc = lane == 0 ? -1 : lane - 1, j = 0;
    unsigned done = 0;
    long long t0 = clock64();
    for (int it = 0; it < steps / 32; ++it) {
        for (int s = 0; s < 32; ++s) {
            const int owner = s;
            const double a = __dsub_rn(bk, ls);
            double q = dg.div_fast(a);
            double xv = __shfl_sync(0xffffffffu, q, owner);
            if (W & 1) {
                if (__ballot_sync(0xffffffffu, !exact_chk(dg, a, q)) >> owner & 1u) {
                    q = __ddiv_rn(a, dg.d);
                    xv = __shfl_sync(0xffffffffu, q, owner);
                }
            }
            if (lane == owner) {
                xm = q;
                done |= 1u;
                if (W & 2) {
                    unsigned long long bits = (unsigned long long)__double_as_longlong(q), e = 1ull << 32;
                    asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(rec + 2 * (size_t)(it * 32 + s) % 8192),
                                 "l"(e | (bits & 0xffffffffull)), "l"(e | (bits >> 32)) : "memory");
                }
            }
            if (W & 4) {
                if (nc == s) {
                    ls = __dadd_rn(0.0, __dmul_rn(nv, xv));
                    ++j;
                    nc = j < 1 ? cols[j] : -1;
                }
            } else if (lane == ((s + 1) & 31)) {
                ls = __dadd_rn(0.0, __dmul_rn(nv, xv));
            }
        }
        nc = lane == 0 ? -1 : lane - 1;
        j = 0;
    }
    long long t1 = clock64();
    if (lane == 0) cyc[W] = (t1 - t0) / steps + (long long)(xm * 0) + done * 0;
}

// The CHAIN engine's warp-redundant fast path (solve_chain.cuh) in isolation: operands in
// smem, all lanes evaluate x_t = (b_t - (ls_t + v_t x_{t-1})) / d_t; W selects the per-step
// publication: 0 none, 1 owner's 16-B relaxed.gpu record store, 2 weak 16-B store, 3 strong
// store + globaltimer trace.
template <int W>
__global__ void k_fast(long long *cyc, int steps, unsigned long long *rec, unsigned long long *tr) {
    __shared__ double f_ls[64], f_b[64], f_v[64], f_d[64], f_r[64];
    __shared__ int f_has[64];
    const int lane = threadIdx.x;
    for (int t = lane; t < 64; t += 32) {
        f_ls[t] = 0.0; f_b[t] = 1.0; f_v[t] = -1.0; f_d[t] = 2.0 + t * 1e-3; f_r[t] = __drcp_rn(f_d[t]); f_has[t] = t > 0;
    }
    __syncwarp();
    double xp = 0.0, xm = 0.0;
    long long t0 = clock64();
    for (int it = 0; it < steps / 32; ++it) {
        double lsv = f_ls[0], bv = f_b[0], vv = f_v[0], dv = f_d[0], rv = f_r[0];
        int hv = f_has[0];
        for (int t = 0; t < 32; ++t) {
            const int tn = min(t + 1, 31);
            const double lsn = f_ls[tn], bn = f_b[tn], vn = f_v[tn], dn = f_d[tn], rn = f_r[tn];
            const int hn = f_has[tn];
            const double u = hv ? __dadd_rn(lsv, __dmul_rn(vv, xp)) : lsv;
            const double a = __dsub_rn(bv, u);
            Diag g;
            g.d = dv;
            g.r = rv;
            double q = g.div_fast(a);
            const unsigned ex = ((unsigned)__double2hiint(a) >> 20) & 0x7FFu;
            if (!(rv != 0.0 && ex - (1023u - 400u) <= 800u)) q = __ddiv_rn(a, dv);
            const bool mine = lane == t;
            xm = mine ? q : xm;
            unsigned long long bits = (unsigned long long)__double_as_longlong(q), e = 1ull << 32;
            const size_t ix = 2 * (size_t)((it * 32 + t) & 4095);
            if (W == 1 || W == 3) {
                if (mine) asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(rec + ix), "l"(e | (bits & 0xffffffffull)), "l"(e | (bits >> 32)) : "memory");
            }
            if (W == 2) {
                if (mine) asm volatile("st.global.v2.u64 [%0], {%1, %2};" ::"l"(rec + ix), "l"(e | (bits & 0xffffffffull)), "l"(e | (bits >> 32)) : "memory");
            }
            if (W == 3 && mine) {
                unsigned long long tt;
                asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tt));
                tr[(it * 32 + t) & 4095] = tt;
            }
            xp = q;
            lsv = lsn, bv = bn, vv = vn, dv = dn, rv = rn, hv = hn;
        }
    }
    long long t1 = clock64();
    if (lane == 0) cyc[W] = (t1 - t0) / steps + (long long)(xm * 0);
}

__global__ void k_lat(long long *cyc, double a0, int iters) {
    double a = a0, b = 1.0000001;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) a = __fma_rn(a, b, 1e-300);
    long long t1 = clock64();
    double c = a0;
    for (int i = 0; i < iters; ++i) c = __dmul_rn(c, b);
    long long t2 = clock64();
    double e = a0;
    for (int i = 0; i < iters; ++i) e = __shfl_sync(0xffffffffu, e, (i + threadIdx.x) & 31);
    long long t3 = clock64();
    double f = a0;
    for (int i = 0; i < iters; ++i) f = __ddiv_rn(f, b);
    long long t4 = clock64();
    if (threadIdx.x == 0) {
        cyc[0] = (t1 - t0) / iters;
        cyc[1] = (t2 - t1) / iters;
        cyc[2] = (t3 - t2) / iters;
        cyc[3] = (t4 - t3) / iters;
        cyc[4] = (long long)(a + c + e + f);
    }
}

int main() {
    double *out;
    long long *cyc, h[8];
    cudaMalloc(&out, 64);
    cudaMalloc(&cyc, 128);
    k_lat<<<1, 32>>>(cyc, 1.5, 10000);
    cudaMemcpy(h, cyc, 40, cudaMemcpyDeviceToHost);
    printf("dependent latency (cycles): DFMA %lld  DMUL %lld  SHFL.64 %lld  __ddiv_rn %lld\n", h[0], h[1], h[2], h[3]);
    const char *names[] = {"verified div (kernel's Diag::div)", "__ddiv_rn", "unchecked Markstein", "verified, slow path branch", "no division", ""};
    k_chain<0><<<1, 32>>>(out, cyc, 32000, 4.0, -1.0, 1.0);
    k_chain<1><<<1, 32>>>(out, cyc, 32000, 4.0, -1.0, 1.0);
    k_chain<2><<<1, 32>>>(out, cyc, 32000, 4.0, -1.0, 1.0);
    k_chain<3><<<1, 32>>>(out, cyc, 32000, 4.0, -1.0, 1.0);
    k_chain<4><<<1, 32>>>(out, cyc, 32000, 4.0, -1.0, 1.0);
    unsigned long long *rec;
    double *xg;
    cudaMalloc(&rec, 16 * 4096);
    cudaMalloc(&xg, 8 * 8192);
    k_chain<5><<<1, 32>>>(out, cyc, 32000, 4.0, -1.0, 1.0, rec, xg);
    k_chain<6><<<1, 32>>>(out, cyc, 32000, 4.0, -1.0, 1.0, rec, xg);
    k_chain<7><<<1, 32>>>(out, cyc, 32000, 4.0, -1.0, 1.0, rec, xg);
    cudaMemcpy(h, cyc, 64, cudaMemcpyDeviceToHost);
    names[5] = "unchecked + smem store";
    const char *n6 = "unchecked + smem + global publish", *n7 = "... + globaltimer trace store";
    printf("chain step, %-36s %lld cycles\n", names[5], h[5]);
    printf("chain step, %-36s %lld cycles\n", n6, h[6]);
    printf("chain step, %-36s %lld cycles\n", n7, h[7]);
    for (int v = 0; v < 5; ++v) printf("chain step, %-36s %lld cycles\n", names[v], h[v]);
    int *cols;
    cudaMalloc(&cols, 64);
    cudaMemset(cols, 0, 64);
    k_step<0><<<1, 32>>>(cyc, 32000, 4.0, rec, cols);
    k_step<1><<<1, 32>>>(cyc, 32000, 4.0, rec, cols);
    k_step<2><<<1, 32>>>(cyc, 32000, 4.0, rec, cols);
    k_step<3><<<1, 32>>>(cyc, 32000, 4.0, rec, cols);
    k_step<4><<<1, 32>>>(cyc, 32000, 4.0, rec, cols);
    k_step<7><<<1, 32>>>(cyc, 32000, 4.0, rec, cols);
    cudaMemcpy(h, cyc, 64, cudaMemcpyDeviceToHost);
    k_fast<0><<<1, 32>>>(cyc + 8, 32000, rec, (unsigned long long *)xg);
    k_fast<1><<<1, 32>>>(cyc + 8, 32000, rec, (unsigned long long *)xg);
    k_fast<2><<<1, 32>>>(cyc + 8, 32000, rec, (unsigned long long *)xg);
    k_fast<3><<<1, 32>>>(cyc + 8, 32000, rec, (unsigned long long *)xg);
    long long hf[4];
    cudaMemcpy(hf, cyc + 8, 32, cudaMemcpyDeviceToHost);
    printf("fast path step: no store %lld | strong rec store %lld | weak store %lld | strong + trace %lld cycles\n",
           hf[0], hf[1], hf[2], hf[3]);
    printf("kernel step: bare %lld | +check/vote %lld | +store %lld | +check+store %lld | +consume %lld | all %lld cycles\n",
           h[0], h[1], h[2], h[3], h[4], h[7]);
    return 0;
}
