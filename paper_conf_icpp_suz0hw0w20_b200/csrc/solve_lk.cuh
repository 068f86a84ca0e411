// solve_lk.cuh -- ENGINE_LEAN_K: the LEAN kernel with K thread-level rows per lane.
//
// Same per-row method as every engine -- Alg.5 Writing-First:
// stream the row, consume the ready prefix of its dependencies in row order,
// divide at the diagonal, publish -- for all-thread-level lower plans.
//
// Why K rows per lane.  In the wide-level regime (c2: 10 levels x 1e5 rows, the
// paper's warp-underutilisation case) the solve is bound by
// how many rows are RESIDENT: rows are dispensed in order (the start ticket), a
// CTA's slot frees only when all its rows published, and the rows of level l+1
// can only be loaded once slots of level l-1 freed.  LEAN holds one row per
// thread (1536 threads per SM at 40 registers, a 227k-row window = 2.3 levels of
// c2); the trace showed new rows entering ~2.3 us (two dependent DRAM round
// trips) after their CTA started, and an event model of that schedule
// (tools/model/sim.py) gains ~25% from a 303k window and ~35% from 454k.  Here
// a lane owns rows r0 + lane + 32k, k < K: the per-row state is ten registers
// (two next dependencies with their values, the cursor, the partial sum), the
// row constants b_i, L_ii, 1/L_ii live in shared memory, and every row's loads
// and polls are independent, so K rows also give K-fold memory-level
// parallelism per thread.
//
// Per pass each unfinished row polls its next TWO dependencies (both values
// preloaded with their columns, so consuming the second never waits on a
// reload); the ready prefix is consumed in row order with separately rounded
// mul and add (bit-identical to Alg.1); a row whose prefix
// reaches the diagonal divides (Diag, the verified Markstein step) and
// publishes.  Forward progress: a lane never blocks on one row (all K are
// polled each pass), rows wait only on earlier rows (same warp, or CTAs that
// took an earlier start ticket), so the earliest unfinished row always advances.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

template <int PROTO, int K, int CT, int MINB>
__global__ void __launch_bounds__(CT, MINB) k_solve_lk(SolveParams p) {
    __shared__ uint32_t s_blk, s_epoch;
    __shared__ double s_b[CT * K], s_d[CT * K], s_r[CT * K];
    constexpr int RPC = CT * K;  // rows per CTA
    const int tid = threadIdx.x;
    const int lane = tid & 31;
    const int wbase = (tid >> 5) * 32 * K + lane;  // CTA-relative row of (this lane, k = 0)
    const uint64_t pol = policy_evict_first();
    // ---- speculative first-level loads for logical block == blockIdx.x
    int rs[K], re[K];
    double bi[K];
    auto load1 = [&](int blk) {
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const int i = blk * RPC + wbase + 32 * k;
            rs[k] = 0, re[k] = 1, bi[k] = 0.0;
            if (i < p.n) {
                rs[k] = ld_stream_i32(p.rowptr + i, pol);
                re[k] = ld_stream_i32(p.rowptr + i + 1, pol);
                bi[k] = ld_stream_f64(p.b + i, pol);
            }
        }
    };
    load1((int)blockIdx.x);
    if (tid == 0) cta_ticket(p, s_blk, s_epoch);
    __syncthreads();
    const uint32_t epoch = s_epoch;
    const int blk = (int)s_blk;
    if (blk != (int)blockIdx.x) load1(blk);  // rare: the ticket assigned another block
    const int row0 = blk * RPC + wbase;
    // ---- second-level loads: L_ii and the first two dependencies with their values
    int c0[K], c1[K], j[K], jd[K];
    double v0[K], v1[K], ls[K];
    unsigned done = 0;
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const bool act = row0 + 32 * k < p.n;
        jd[k] = re[k] - 1;
        const double dv = act ? ld_stream_f64(p.val + jd[k], pol) : 1.0;
        const bool h0 = act && rs[k] < jd[k], h1 = act && rs[k] + 1 < jd[k];
        c0[k] = h0 ? ld_stream_i32(p.colidx + rs[k], pol) : -1;
        v0[k] = h0 ? ld_stream_f64(p.val + rs[k], pol) : 0.0;
        c1[k] = h1 ? ld_stream_i32(p.colidx + rs[k] + 1, pol) : -1;
        v1[k] = h1 ? ld_stream_f64(p.val + rs[k] + 1, pol) : 0.0;
        j[k] = rs[k] + 2;
        ls[k] = 0.0;
        Diag dg;
        dg.init(dv);
        const int t = wbase + 32 * k;
        s_b[t] = bi[k];
        s_d[t] = dg.d;
        s_r[t] = dg.r;
        if (!act) done |= 1u << k;
    }
    Cta nocta;
    nocta.R0 = nocta.R1 = 0;
    nocta.xc = nullptr;
    nocta.xc_s = 0;
    p.local = 0;  // no in-CTA x copy in this engine
    // the next two entries after a consumed prefix of 1 or 2
    auto refill = [&](int k, int used) {
        if (used == 2) {
            const bool h0 = j[k] < jd[k], h1 = j[k] + 1 < jd[k];
            c0[k] = h0 ? ld_stream_i32(p.colidx + j[k], pol) : -1;
            v0[k] = h0 ? ld_stream_f64(p.val + j[k], pol) : 0.0;
            c1[k] = h1 ? ld_stream_i32(p.colidx + j[k] + 1, pol) : -1;
            v1[k] = h1 ? ld_stream_f64(p.val + j[k] + 1, pol) : 0.0;
            j[k] += 2;
        } else {
            const bool h1 = j[k] < jd[k];
            c0[k] = c1[k];
            v0[k] = v1[k];
            c1[k] = h1 ? ld_stream_i32(p.colidx + j[k], pol) : -1;
            v1[k] = h1 ? ld_stream_f64(p.val + j[k], pol) : 0.0;
            j[k] += 1;
        }
    };
    auto finish = [&](int k) {  // Alg.5 l.13-16: x_i = (b_i - left_sum) / L_ii, publish
        const int t = wbase + 32 * k;
        Diag dg;
        dg.d = s_d[t];
        dg.r = s_r[t];
        publish<PROTO>(p, nocta, row0 + 32 * k, dg.div(__dsub_rn(s_b[t], ls[k])), epoch);
        done |= 1u << k;
    };
    uint32_t backoff = p.backoff_min, idle = 0;
    while (true) {
        bool prog = false;
        unsigned long long a0[K], a1[K], b0[K], b1[K];
#pragma unroll
        for (int k = 0; k < K; ++k) {  // issue every row's polls first: K x 2 loads in flight
            a0[k] = a1[k] = b0[k] = b1[k] = 0;
            if (!(done >> k & 1u) && c0[k] >= 0) {
                poll1<PROTO>(p, c0[k], a0[k], a1[k]);
                if (c1[k] >= 0) poll1<PROTO>(p, c1[k], b0[k], b1[k]);
            }
        }
#pragma unroll
        for (int k = 0; k < K; ++k) {
            if (done >> k & 1u) continue;
            if (c0[k] < 0) {  // no dependency left (diagonal-only row)
                finish(k);
                prog = true;
                continue;
            }
            if (!ready1<PROTO>(a0[k], a1[k], epoch)) continue;
            ls[k] = __dadd_rn(ls[k], __dmul_rn(v0[k], value1<PROTO>(p, c0[k], a0[k], a1[k])));
            int used = 1;
            if (c1[k] >= 0 && ready1<PROTO>(b0[k], b1[k], epoch)) {
                ls[k] = __dadd_rn(ls[k], __dmul_rn(v1[k], value1<PROTO>(p, c1[k], b0[k], b1[k])));
                used = 2;
            }
            refill(k, used);
            prog = true;
            if (c0[k] < 0) finish(k);  // the prefix reached the diagonal (Alg.5 l.12)
        }
        if (!__ballot_sync(FULL, done != (1u << K) - 1u)) break;
        if (__ballot_sync(FULL, prog)) {
            backoff = p.backoff_min;
            idle = 0;
            continue;
        }
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
            if (__shfl_sync(FULL, ab, 0)) break;
        }
    }
}

}  // namespace sptrsv_dev
