// solve_k.cuh -- K rows per lane: coarsened thread-level Writing-First.
//
// k_solve_k<PROTO, K> is the one-shot engine for all-thread-level plans with
// each lane owning K rows, i_k = r0 + lane + 32k (k = 0..K-1), so a warp task
// covers 32K consecutive rows.  It is Alg.5 per row: every
// pass, each of the lane's unfinished rows polls its next dependency, consumes
// it if ready (row order, separately rounded mul/add -- bit-identical to
// Alg.1) and solves + publishes when it reaches the diagonal.  The K polls of a
// lane are in flight together, and the number of rows in flight per resident
// thread grows K-fold -- the lever for configurations whose wavefront needs
// more concurrently active rows than the GPU has threads.
// Everything else (CTA ticket, epoch, FLAGS/FUSED protocol, in-CTA shared-memory
// x copy, lean wait loop) is the one-shot engine's.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

// Shared memory per warp for K rows per lane: rowptr [32K+1], b [32K], 1/L_ii [32K],
// and the CSR slice [kSliceK * K] (colidx + val).
constexpr int kSliceK = 112;  // staged entries per 32 rows (3.5 per row)

__host__ __device__ constexpr int k_warp_smem_bytes(int K) {
    return ((4 * (32 * K + 1) + 15) / 16) * 16 + 8 * 32 * K + 8 * 32 * K + kSliceK * K * (4 + 8);
}

template <int PROTO, int K>
__device__ __forceinline__ bool thread_rows_k(const SolveParams &p, const Cta &cta, int r0, uint32_t epoch,
                                              int lane, unsigned char *wsm, uint64_t pol) {
    constexpr int RT = 32 * K;
    constexpr int ECAP = kSliceK * K;
    int32_t *s_rp = reinterpret_cast<int32_t *>(wsm);
    double *s_b = reinterpret_cast<double *>(wsm + ((4 * (RT + 1) + 15) / 16) * 16);
    double *s_r = s_b + RT;
    double *s_val = s_r + RT;
    int32_t *s_col = reinterpret_cast<int32_t *>(s_val + ECAP);
    const int rows = min(RT, p.n - r0);
    // ---- stage rowptr, b (coalesced), then the warp's contiguous CSR slice
#pragma unroll
    for (int m = 0; m <= K; ++m) {
        const int idx = lane + 32 * m;
        if (idx <= rows) s_rp[idx] = ld_stream_i32(p.rowptr + r0 + idx, pol);
    }
#pragma unroll
    for (int m = 0; m < K; ++m) {
        const int idx = lane + 32 * m;
        if (idx < rows) s_b[idx] = ld_stream_f64(p.b + r0 + idx, pol);
    }
    __syncwarp();
    const int base = s_rp[0];
    const int len = s_rp[rows] - base;
    const bool staged = p.stage && len <= ECAP;  // warp-uniform
    if (staged) {
#pragma unroll 4
        for (int e = lane; e < len; e += 32) {
            s_col[e] = ld_stream_i32(p.colidx + base + e, pol);
            s_val[e] = ld_stream_f64(p.val + base + e, pol);
        }
        __syncwarp();
    }
    auto col_at = [&](int jj) -> int { return staged ? s_col[jj - base] : ld_stream_i32(p.colidx + jj, pol); };
    auto val_at = [&](int jj) -> double { return staged ? s_val[jj - base] : ld_stream_f64(p.val + jj, pol); };
    const int R0 = p.local ? cta.R0 : 0x7fffffff;
    // ---- per-row state (registers): entry cursor, diagonal index, next dependency, partial sum
    int j[K], jd[K], nc[K];
    double nv[K], ls[K];
    unsigned done = 0;
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const int idx = lane + 32 * k;
        const bool a = idx < rows;
        j[k] = a ? s_rp[idx] : 0;
        jd[k] = a ? s_rp[idx + 1] - 1 : 0;
        nc[k] = (a && j[k] < jd[k]) ? col_at(j[k]) : -1;
        nv[k] = (a && j[k] < jd[k]) ? val_at(j[k]) : 0.0;
        ls[k] = 0.0;
        if (!a) done |= 1u << k;
        if (a) {  // 1/L_ii, off the critical path (see Diag)
            Diag dg;
            dg.init(val_at(jd[k]));
            s_r[idx] = dg.r;
        }
    }
    const unsigned all = (1u << K) - 1u;
    auto publish_k = [&](int k) {
        const int idx = lane + 32 * k;
        Diag dg;
        dg.d = val_at(jd[k]);
        dg.r = s_r[idx];
        publish<PROTO>(p, cta, r0 + idx, dg.div(__dsub_rn(s_b[idx], ls[k])), epoch);
        done |= 1u << k;
    };
    auto advance = [&](int k) {
        ++j[k];
        nc[k] = j[k] < jd[k] ? col_at(j[k]) : -1;
        nv[k] = j[k] < jd[k] ? val_at(j[k]) : 0.0;
    };
    uint32_t backoff = p.backoff_min, idle = 0;
    while (true) {
        // ---- A. one global poll per unfinished row whose next dependency is in another CTA
        unsigned gm = 0;
        unsigned long long w0[K], w1[K];
#pragma unroll
        for (int k = 0; k < K; ++k) {
            w0[k] = 0;
            w1[k] = 0;
            if (!(done >> k & 1u) && nc[k] >= 0 && nc[k] < R0) {
                gm |= 1u << k;
                poll1<PROTO>(p, nc[k], w0[k], w1[k]);
            }
        }
        bool prog = false;
        // ---- B. local rounds over the rows whose next dependency is in this CTA (or the diagonal)
        if (__ballot_sync(FULL, (done | gm) != all)) {
            while (true) {
                bool lp = false;
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    if ((done | gm) >> k & 1u) continue;
                    if (nc[k] < 0) {
                        publish_k(k);
                        lp = true;
                    } else {
                        const unsigned long long v =
                            ld_volatile_smem_u64_at(cta.xc_s + 8u * (unsigned)(nc[k] - cta.R0));
                        if (v != kSentinel) {
                            if (p.trace) p.trace[p.n + r0 + lane + 32 * k] = globaltimer_ns();
                            ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], __longlong_as_double((long long)v)));
                            advance(k);
                            if (nc[k] < 0) publish_k(k);
                            lp = true;
                        }
                    }
                }
                if (!__ballot_sync(FULL, lp)) break;
                prog = true;
            }
        }
        // ---- C. consume the global polls
#pragma unroll
        for (int k = 0; k < K; ++k) {
            if (!(gm >> k & 1u)) continue;
            if (ready1<PROTO>(w0[k], w1[k], epoch)) {
                if (p.trace) p.trace[p.n + r0 + lane + 32 * k] = globaltimer_ns();
                ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], value1<PROTO>(p, nc[k], w0[k], w1[k])));
                advance(k);
                if (nc[k] < 0) publish_k(k);
                prog = true;
            }
        }
        if (!__ballot_sync(FULL, done != all)) break;
        if (__ballot_sync(FULL, prog)) {
            backoff = p.backoff_min;
            idle = 0;
            continue;
        }
        // ---- D. lean wait: poll each unfinished row's blocking dependency; consume what is ready
        while (true) {
            if (backoff) nanosleep_ns(backoff);
            backoff = min(max(backoff * 2u, 32u), p.backoff_max);
            if ((++idle & 63u) == 0) {
                uint32_t ab = 0;
                if (lane == 0) {
                    if (p.spin_limit && idle >= p.spin_limit) {
                        atomicCAS(&p.st->error.v, 0u, 1u);
                        st_relaxed_u32(&p.st->abort.v, 1u);
                    }
                    ab = ld_relaxed_u32(&p.st->abort.v);
                }
                if (__shfl_sync(FULL, ab, 0)) return false;
            }
            bool rdy = false;
#pragma unroll
            for (int k = 0; k < K; ++k) {
                if (done >> k & 1u) continue;
                double xv = 0.0;
                bool r;
                if (nc[k] < R0) {
                    unsigned long long a0, a1;
                    poll1<PROTO>(p, nc[k], a0, a1);
                    r = ready1<PROTO>(a0, a1, epoch);
                    if (r) xv = value1<PROTO>(p, nc[k], a0, a1);
                } else {
                    const unsigned long long v = ld_volatile_smem_u64_at(cta.xc_s + 8u * (unsigned)(nc[k] - cta.R0));
                    r = v != kSentinel;
                    xv = __longlong_as_double((long long)v);
                }
                if (r) {
                    if (p.trace) p.trace[p.n + r0 + lane + 32 * k] = globaltimer_ns();
                    ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], xv));
                    advance(k);
                    if (nc[k] < 0) publish_k(k);
                    rdy = true;
                }
            }
            if (__ballot_sync(FULL, rdy)) {
                backoff = p.backoff_min;
                idle = 0;
                break;
            }
        }
        if (!__ballot_sync(FULL, done != all)) break;
    }
    __syncwarp();
    return true;
}

template <int PROTO, int K>
__global__ void __launch_bounds__(256) k_solve_k(SolveParams p) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint32_t s_blk, s_epoch;
    constexpr int RT = 32 * K;
    const int warps = blockDim.x >> 5;
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    if (threadIdx.x == 0) cta_ticket(p, s_blk, s_epoch);
    __syncthreads();
    const uint32_t epoch = s_epoch;
    const int blk = (int)s_blk;
    const uint64_t pol = policy_evict_first();
    Cta cta;
    cta.xc = reinterpret_cast<unsigned long long *>(smem);
    cta.xc_s = (unsigned)__cvta_generic_to_shared(cta.xc);
    cta.R0 = blk * warps * RT;
    cta.R1 = min(p.n, cta.R0 + warps * RT);
    if (p.local) {
        for (int k = threadIdx.x; k < cta.R1 - cta.R0; k += blockDim.x) cta.xc[k] = kSentinel;
        __syncthreads();
    }
    const int r0 = cta.R0 + warp * RT;
    unsigned char *wsm = smem + (size_t)warps * RT * 8 + (size_t)warp * k_warp_smem_bytes(K);
    if (r0 < p.n) thread_rows_k<PROTO, K>(p, cta, r0, epoch, lane, wsm, pol);
}

}  // namespace sptrsv_dev
