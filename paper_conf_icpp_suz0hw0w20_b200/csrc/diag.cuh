// diag.cuh -- diagnostics outside the timed solve: GPU level analysis (SURVEY
// row a10) and the flag-hop microbenchmark (t_hop of the latency bound).
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

// ---------------------------------------------------------------- levels (diagnostic)
//
// lvl[i] = level(i) + 1 once known, 0 before.  The value IS the
// message, so a relaxed poll suffices (no second location is read).
// level(i) = max over dependencies of lvl[j] (= 1 + level(j)), 0 without any.
__global__ void __launch_bounds__(256) k_levels(const int32_t *__restrict__ rowptr,
                                                const int32_t *__restrict__ colidx, uint32_t *lvl,
                                                SolveState *st, int32_t n) {
    __shared__ uint32_t s_blk;
    if (threadIdx.x == 0) s_blk = atomicAdd(&st->lticket.v, 1u);
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int r0 = ((int)s_blk * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32;
    if (r0 >= n) return;
    const int i = r0 + lane;
    const bool act = i < n;
    int j = 0, jd = 0;
    if (act) {
        j = rowptr[i];
        jd = rowptr[i + 1] - 1;
    }
    uint32_t cur = 0;
    bool done = !act;
    uint32_t backoff = 0;
    while (true) {
        bool prog = false;
        if (!done) {
            const int m = min(kU, jd - j);
            uint32_t f[kU];
#pragma unroll
            for (int k = 0; k < kU; ++k) f[k] = (k < m) ? ld_relaxed_u32(lvl + colidx[j + k]) : 0u;
            int q = 0;
#pragma unroll
            for (int k = 0; k < kU; ++k)
                if (q == k && k < m && f[k] != 0u) {
                    q = k + 1;
                    cur = max(cur, f[k]);
                }
            j += q;
            prog = q > 0;
            if (j == jd) {
                st_relaxed_u32(lvl + i, cur + 1u);
                done = true;
                prog = true;
            }
        }
        if (!__ballot_sync(FULL, !done)) break;
        if (__ballot_sync(FULL, prog)) {
            backoff = 0;
        } else {
            if (backoff) nanosleep_ns(backoff);
            backoff = backoff ? min(backoff * 2u, 1024u) : 32u;
        }
    }
}

__global__ void k_level_finish(const uint32_t *__restrict__ lvl, int32_t *level_out,
                               int32_t *counts, int32_t *nlevels, int32_t n) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const bool act = i < n;
    const int lv = act ? (int)lvl[i] - 1 : -1;
    if (act && level_out) level_out[i] = lv;
    // warp-aggregated histogram: lanes with the same level add once
    const unsigned am = __ballot_sync(FULL, act);
    if (act) {
        const unsigned peers = __match_any_sync(am, lv);
        if (counts && (__ffs(peers) - 1) == (threadIdx.x & 31)) atomicAdd(counts + lv, __popc(peers));
    }
    int mx = lv;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) mx = max(mx, __shfl_xor_sync(FULL, mx, off));
    if ((threadIdx.x & 31) == 0 && mx >= 0) atomicMax(nlevels, mx + 1);
}

// ---------------------------------------------------------------- flag-hop microbenchmark
//
// Two single-thread CTAs (normally on different SMs) bounce `iters` messages.
// Each message = an x value + its flag, published and consumed exactly as the
// solve does it (protocol 0), or with relaxed polls + fence.acq_rel (1), or
// value-as-flag (2).  Single-CTA probes: 3 = dependent ld.relaxed.gpu chain
// (L2 round trip), 4 = st x + st.release flag pairs (publish cost).
// out[0] = elapsed ns on CTA 0, out[1] = elapsed SM cycles on CTA 0.
__global__ void k_pingpong(uint32_t *flags, double *xs, int iters, int protocol,
                           unsigned long long *out, double *sink) {
    if (threadIdx.x != 0) return;
    const int me = blockIdx.x;
    uint32_t *myf = flags + me * 32;
    uint32_t *of = flags + (1 - me) * 32;
    double *myx = xs + me * 16;
    double *ox = xs + (1 - me) * 16;
    double acc = 0.0;
    const uint64_t t0 = globaltimer_ns();
    const long long c0 = clock64();
    if (protocol >= 3) {
        if (me == 0) {
            if (protocol == 5) {  // dependent IEEE fp64 divisions
                double v = 1.5, d = 1.0000001;
                for (int k = 0; k < iters; ++k) v = __ddiv_rn(v + 1.0, d);
                acc = v;
            } else if (protocol == 6) {  // dependent DFMA chain
                double v = 1.5;
                for (int k = 0; k < iters; ++k) v = fma(v, 0.999999, 1e-7);
                acc = v;
            } else if (protocol == 7) {  // shared-memory store -> volatile load round trip
                __shared__ unsigned long long sm[64];
                unsigned long long v = 0;
                for (int k = 0; k < iters; ++k) {
                    asm volatile("st.volatile.shared.u64 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(sm + (v & 1))), "l"(v + 1) : "memory");
                    asm volatile("ld.volatile.shared.u64 %0, [%1];" : "=l"(v) : "r"((unsigned)__cvta_generic_to_shared(sm + (v & 1))) : "memory");
                }
                acc = (double)v;
            } else if (protocol == 3) {
                uint32_t v = 0;
                for (int k = 0; k < iters; ++k) v = ld_relaxed_u32(flags + 64 + (v & 1u));
                acc = v;
            } else {
                for (int k = 1; k <= iters; ++k) {
                    myx[0] = (double)k;
                    st_release_u32(myf, (uint32_t)k);
                }
            }
        }
    } else {
        for (int k = 1; k <= iters; ++k) {
            const bool send_first = (me == 0);
            for (int phase = 0; phase < 2; ++phase) {
                const bool send = (phase == 0) == send_first;
                if (send) {
                    if (protocol == 2) {
                        st_relaxed_f64(myx, (double)k);
                    } else {
                        myx[0] = (double)k;
                        st_release_u32(myf, (uint32_t)k);
                    }
                } else {
                    if (protocol == 0) {
                        while (ld_acquire_u32(of) != (uint32_t)k) {}
                        acc += ld_relaxed_f64(ox);
                    } else if (protocol == 1) {
                        while (ld_relaxed_u32(of) != (uint32_t)k) {}
                        fence_acq_rel_gpu();
                        acc += ld_relaxed_f64(ox);
                    } else {
                        double v;
                        while ((v = ld_relaxed_f64(ox)) != (double)k) {}
                        acc += v;
                    }
                }
            }
        }
    }
    const long long c1 = clock64();
    const uint64_t t1 = globaltimer_ns();
    if (me == 0) {
        out[0] = t1 - t0;
        out[1] = (unsigned long long)(c1 - c0);
    }
    sink[me] = acc;
}

// ---------------------------------------------------------------- placement-controlled hop (t_hop per die pair)
// One CTA per SM: the launch requests more than half of an SM's shared memory, so the grid of
// #SMs CTAs lands one per SM, all co-resident.  k_smids records which SM each CTA landed on;
// in k_pingpong_sm the CTAs on SMs sm_a and sm_b ping-pong `iters` rounds through the solve's
// protocol (0: st.release flag / ld.acquire poll + relaxed x load; 1: FUSED 16-byte epoch
// record, relaxed store / relaxed poll) and the others exit at once.  The one-way hop between
// a given pair of SMs is then independent of where the scheduler puts CTAs.
__device__ __forceinline__ unsigned smid_u32() {
    unsigned s;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
    return s;
}

__global__ void k_smids(int32_t *out) {
    extern __shared__ unsigned char pad_[];
    if (threadIdx.x == 0) {
        pad_[0] = 0;
        out[blockIdx.x] = (int32_t)smid_u32();
    }
}

__global__ void k_pingpong_sm(unsigned long long *rec, uint32_t *flags, double *xs, int iters, int protocol,
                              int sm_a, int sm_b, unsigned long long *out, double *sink) {
    extern __shared__ unsigned char pad_[];
    if (threadIdx.x != 0) return;
    pad_[0] = 0;
    const int s = (int)smid_u32();
    const int me = s == sm_a ? 0 : s == sm_b ? 1 : -1;
    if (me < 0) return;
    unsigned long long *myr = rec + 16 * me, *orr = rec + 16 * (1 - me);  // 128 B apart
    uint32_t *myf = flags + 32 * me, *of = flags + 32 * (1 - me);
    double *myx = xs + 16 * me, *ox = xs + 16 * (1 - me);
    double acc = 0.0;
    const uint64_t t0 = globaltimer_ns();
    for (int k = 1; k <= iters; ++k) {
        for (int phase = 0; phase < 2; ++phase) {
            const bool send = (phase == 0) == (me == 0);
            if (send) {
                if (protocol == 0) {
                    myx[0] = (double)k;
                    st_release_u32(myf, (uint32_t)k);
                } else {
                    const unsigned long long bits = (unsigned long long)__double_as_longlong((double)k);
                    const unsigned long long e = (unsigned long long)k << 32;
                    st_relaxed_v2_u64(myr, e | (bits & 0xffffffffull), e | (bits >> 32));
                }
            } else {
                if (protocol == 0) {
                    while (ld_acquire_u32(of) != (uint32_t)k) {}
                    acc += ld_relaxed_f64(ox);
                } else {
                    unsigned long long a, b;
                    do {
                        ld_relaxed_v2_u64(orr, a, b);
                    } while ((uint32_t)(a >> 32) != (uint32_t)k || (uint32_t)(b >> 32) != (uint32_t)k);
                    acc += __longlong_as_double((long long)((a & 0xffffffffull) | (b << 32)));
                }
            }
        }
    }
    const uint64_t t1 = globaltimer_ns();
    if (me == 0) out[0] = t1 - t0;
    sink[me] = acc;
}

}  // namespace sptrsv_dev
