// solve_tri.cuh -- SURVEY row f4, hybrid plans: one warp per long row (Alg.3,
// PAPER.md:120-149, the sec.4.4 hybrid's long-row kernel) and one lane
// per short row (Alg.5 via lean_rows) for UPPER and/or UNIT-diagonal handles whose plan
// has warp-level rows.  All-thread-level f4 plans run in k_solve_lean.
//
// Logical row r (start-ticket order) is row i = r (lower) or i = n-1-r (upper), so the
// ticket order is a topological order either way.  The off-diagonals [lo, hi) are fed to
// warp_row (solve.cuh) through an index map that walks them earliest-solved first
// (ascending column for lower, DESCENDING for upper, G25); lane partial sums and
// the butterfly make the result equal the substitution within the warp-mode bound
// (parity), exactly as for lower warp rows.  UNIT: the divisor is 1.0, which
// the verified division returns exactly (b_i - sum).
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"
#include "solve_lean.cuh"

namespace sptrsv_dev {

constexpr int kTriWarpCta = 64;  // 2 warps: the CTA size measured best for warp plans (c4)

// Warp-level row: logical row r -> row i; off-diagonals fed earliest-solved first.
template <int PROTO, bool UPPER, bool UNIT>
__device__ __forceinline__ void tri_warp_row(SolveParams &p, int r, uint32_t epoch, int lane, uint64_t pol) {
    const int i = UPPER ? p.n - 1 - r : r;
    const int rs = ld_stream_i32(p.rowptr + i, pol);
    const int re = ld_stream_i32(p.rowptr + i + 1, pol);
    const int lo = (UPPER && !UNIT) ? rs + 1 : rs;
    const int hi = (UPPER || UNIT) ? re : re - 1;
    double bi = 0.0, dv = 1.0;
    if (lane == 0) {
        bi = ld_b(p, i, pol);
        if (!UNIT) dv = ld_stream_f64(p.val + (UPPER ? rs : re - 1), pol);
    }
    Cta nocta;
    nocta.R0 = nocta.R1 = 0;
    nocta.xc = nullptr;
    nocta.xc_s = 0;
    // warp_row walks t in [0, hi - lo) (its "diagonal" sits at t = hi - lo)
    auto at = [&](int t) { return UPPER ? hi - 1 - t : lo + t; };
    warp_row<PROTO>(p, nocta, i, 0, hi - lo + 1, bi, dv, epoch, lane,
                    [&](int t) -> int { return ld_stream_i32(p.colidx + at(t), pol); },
                    [&](int t) -> double { return ld_stream_f64(p.val + at(t), pol); });
}

// Sub-warp rows (the thread-vs-warp granularity of sec.4.4): W lanes
// per row, 32 / W consecutive logical rows r0 .. r0 + 32/W - 1 per warp task.  Each row is Alg.3 on
// a W-lane segment: sub-lane sl consumes the off-diagonals at walk positions sl, sl + W, ... in
// order as they become ready (entries fed earliest-solved first, as in warp_row); once every lane
// of a segment is through, a __shfl_xor tree sums the segment's W partials, and the row's leader
// lane adds the last off-diagonal (its nearest dependency, polled on its own --
// SPTRSV_OPT_WARP_SPLIT_LAST), divides and publishes.  Rows of one task may depend on each other
// (consecutive rows), so nothing blocks: like Alg.5's Writing-First every pass polls, consumes what
// is ready and moves on, and each segment reduces and publishes the moment it can (Challenge 1,
// PAPER.md:226).  A fixed, data-independent summation order (deterministic; within the warp-mode
// bound of DESIGN.md).
constexpr int kSubB = 4;  // entries per lane in flight (one batch)

template <int PROTO, int W, bool UPPER, bool UNIT>
__device__ __forceinline__ void subwarp_rows(SolveParams &p, int r0, uint32_t epoch, int lane, uint64_t pol) {
    const int sl = lane & (W - 1);
    const int r = r0 + lane / W;
    const bool act = r < p.n;
    const bool leader = act && sl == 0;
    const int i = UPPER ? p.n - 1 - r : r;
#ifdef SPTRSV_MEASURE_ROWSTART  // measurement builds only (tools/trace_polls.py): task start per row
    if (p.trace && leader) p.trace[2 * (size_t)p.n + i] = globaltimer_ns();
#endif
    int rs = 0, re = 0;
    if (act) {
        rs = ld_stream_i32(p.rowptr + i, pol);
        re = ld_stream_i32(p.rowptr + i + 1, pol);
    }
    const int lo = (UPPER && !UNIT) ? rs + 1 : rs;
    const int hi = (UPPER || UNIT) ? re : re - 1;
    const int len = act ? hi - lo : 0;  // off-diagonals of the row
    auto at = [&](int t) { return UPPER ? hi - 1 - t : lo + t; };
    const bool has_last = p.split_last && len > 0;
    const int m = has_last ? len - 1 : len;  // entries in the lane-strided part
    // the leader's row constants and last dependency, loaded up front (off the critical path)
    double bi = 0.0, dv = 1.0, v_last = 0.0;
    int c_last = 0;
    if (leader) {
        bi = ld_b(p, i, pol);
        if (!UNIT) dv = ld_stream_f64(p.val + (UPPER ? rs : re - 1), pol);
        if (has_last) {
            c_last = ld_stream_i32(p.colidx + at(len - 1), pol);
            v_last = ld_stream_f64(p.val + at(len - 1), pol);
        }
    }
    Diag dg;
    dg.init(dv);
    // this lane's batch: walk positions sl + W * (jb + k), k < mm; q of them consumed
    int c[kSubB];
    double v[kSubB];
    int jb = 0, mm = 0, q = 0;
    auto load_batch = [&]() {
        mm = 0;
        q = 0;
#pragma unroll
        for (int k = 0; k < kSubB; ++k) {
            const int tt = sl + W * (jb + k);
            c[k] = 0;
            v[k] = 0.0;
            if (tt < m) {
                c[k] = ld_stream_i32(p.colidx + at(tt), pol);
                v[k] = ld_stream_f64(p.val + at(tt), pol);
                mm = k + 1;
            }
        }
    };
    load_batch();
    double acc = 0.0, tot = 0.0;
    bool lane_done = mm == 0, reduced = false, published = !leader;
    const unsigned segmask = W == 32 ? FULL : ((1u << W) - 1u) << (lane & ~(W - 1));
    uint32_t backoff = p.backoff_min, idle = 0;
#ifdef SPTRSV_MEASURE_POLLS
    unsigned long long np_ = 0, tl_ = 0;
#endif
    while (true) {
        bool prog = false;
        if (!lane_done) {  // poll the batch, consume its ready prefix in order
            unsigned long long w0[kSubB], w1[kSubB];
#pragma unroll
            for (int k = 0; k < kSubB; ++k) {
                w0[k] = 0;
                w1[k] = 0;
                if (k >= q && k < mm) poll1<PROTO>(p, c[k], w0[k], w1[k]);
            }
            int nq = q;
#pragma unroll
            for (int k = 0; k < kSubB; ++k)
                if (nq == k && k < mm && ready1<PROTO>(w0[k], w1[k], epoch)) nq = k + 1;
#pragma unroll
            for (int k = 0; k < kSubB; ++k)
                if (k >= q && k < nq) acc = __dadd_rn(acc, __dmul_rn(v[k], value1<PROTO>(p, c[k], w0[k], w1[k])));
            prog = nq > q;
            q = nq;
            if (q == mm) {  // batch through: the next one, or this lane is done
                jb += kSubB;
                load_batch();
                lane_done = mm == 0;
            }
        }
        // segments whose W lanes are all through: the lane tree (all lanes run it, only the
        // newly complete segments keep the result)
        const unsigned dn = __ballot_sync(FULL, lane_done);
        const bool complete = (dn & segmask) == segmask;
        if (__any_sync(FULL, complete && !reduced)) {
            double t = acc;
#pragma unroll
            for (int off = W / 2; off > 0; off >>= 1) t = __dadd_rn(t, __shfl_xor_sync(FULL, t, off));
            if (complete && !reduced) {
                tot = t;
                reduced = true;
                prog = true;
            }
        }
        // a reduced row's leader: its last (nearest) dependency, then divide and publish
        if (!published && reduced) {
            bool go = true;
            if (has_last) {
                unsigned long long w0, w1;
#ifdef SPTRSV_MEASURE_POLLS  // measurement builds only (tools/trace_polls.py): wait start, last poll, polls
                if (p.trace) {
#ifndef SPTRSV_MEASURE_ROWSTART
                    if (np_ == 0) p.trace[2 * (size_t)p.n + i] = globaltimer_ns();
#endif
                    tl_ = globaltimer_ns();
                }
                ++np_;
#endif
                poll1<PROTO>(p, c_last, w0, w1);
                go = ready1<PROTO>(w0, w1, epoch);
                if (go) tot = __dadd_rn(tot, __dmul_rn(v_last, value1<PROTO>(p, c_last, w0, w1)));
            }
            if (go) {
                if (p.trace) p.trace[p.n + i] = globaltimer_ns();
#ifdef SPTRSV_MEASURE_POLLS
                if (p.trace && has_last) p.trace[3 * (size_t)p.n + 3 + i] = (np_ << 40) | (tl_ & ((1ull << 40) - 1));
#endif
                Cta nocta;
                nocta.R0 = nocta.R1 = 0;
                nocta.xc = nullptr;
                nocta.xc_s = 0;
                const double a = __dsub_rn(bi, tot);
                publish<PROTO>(p, nocta, i, UNIT ? a : dg.div(a), epoch);
                published = true;
                prog = true;
            }
        }
        if (!__any_sync(FULL, !published)) break;
        if (__any_sync(FULL, prog)) {
            backoff = p.backoff_min;
            idle = 0;
            continue;
        }
        if (backoff) nanosleep_ns(backoff);
        // rows waiting only on their last dependency keep the short sleeps of warp rows
        backoff = min(max(backoff * 2u, 32u),
                      (p.split_last == 2 && !__any_sync(FULL, !lane_done)) ? 32u : p.backoff_max);
        if ((++idle & 63u) == 0) {
            uint32_t ab = 0;
            if (lane == 0) {
                if (p.spin_limit && idle >= p.spin_limit) {
                    atomicCAS(&p.st->error.v, 0u, kErrTimeout);
                    st_relaxed_u32(&p.st->abort.v, 1u);
                }
                ab = ld_relaxed_u32(&p.st->abort.v);
            }
            if (__shfl_sync(FULL, ab, 0)) return;
        }
    }
}

template <int PROTO, bool UPPER, bool UNIT>
__device__ __forceinline__ void subwarp_task(SolveParams &p, int r0, int w, uint32_t epoch, int lane, uint64_t pol) {
    switch (w) {
        case 2: subwarp_rows<PROTO, 2, UPPER, UNIT>(p, r0, epoch, lane, pol); break;
        case 4: subwarp_rows<PROTO, 4, UPPER, UNIT>(p, r0, epoch, lane, pol); break;
        case 8: subwarp_rows<PROTO, 8, UPPER, UNIT>(p, r0, epoch, lane, pol); break;
        default: subwarp_rows<PROTO, 16, UPPER, UNIT>(p, r0, epoch, lane, pol); break;
    }
}

// PLAN_WARP: task t = logical row t.  PLAN_LIST: tasks[t] >= 0 is a 32-row thread-level
// group starting at that logical row (one row per lane, lean_rows), ~row a warp-level row;
// the list is in logical (ticket) order, built by build_plan over reversed rows for UPPER.
template <int PROTO, bool UPPER, bool UNIT, int PLAN, int CT = kTriWarpCta>
__global__ void __launch_bounds__(CT) k_solve_tri_warp(SolveParams p) {
    __shared__ uint32_t s_blk, s_epoch;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        cta_ticket(p, s_blk, s_epoch);
        if (p.bflag) {  // sptrsv_solve_host: the b chunks of this CTA's tasks' (physical) rows
            int lo = p.n, hi = 0;  // logical row range of the CTA's tasks
            for (int t = (int)s_blk * (CT / 32); t < min(p.n_tasks, ((int)s_blk + 1) * (CT / 32)); ++t) {
                int r0 = t, r1 = t + 1;
                if (PLAN == PLAN_LIST) {
                    const int v = p.tasks[t];
                    const int w = p.task_w[t];
                    r0 = v >= 0 ? v : ~v;
                    r1 = min(p.n, v >= 0 ? v + 32 : r0 + (w > 0 && w < 32 ? 32 / w : 1));
                }
                lo = min(lo, r0);
                hi = max(hi, r1);
            }
            if (lo < hi) wait_b_chunks(p, UPPER ? p.n - hi : lo, UPPER ? p.n - lo : hi);
        }
    }
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const int task = (int)s_blk * (CT / 32) + warp;
    if (task >= p.n_tasks) return;
    const uint64_t pol = policy_evict_first();
    p.local = 0;
    if (PLAN == PLAN_WARP) {
        tri_warp_row<PROTO, UPPER, UNIT>(p, task, epoch, lane, pol);
        return;
    }
    const int t = __ldg(p.tasks + task);
    if (t < 0) {
        const int w = __ldg(p.task_w + task);
        if (w == 32)
            tri_warp_row<PROTO, UPPER, UNIT>(p, ~t, epoch, lane, pol);
        else
            subwarp_task<PROTO, UPPER, UNIT>(p, ~t, w, epoch, lane, pol);
        return;
    }
    const int r = t + lane;
    const bool act = r < p.n;
    const int i = UPPER ? p.n - 1 - r : r;
    int rs = 0, re = 1;
    double bi = 0.0;
    if (act) {
        rs = ld_stream_i32(p.rowptr + i, pol);
        re = ld_stream_i32(p.rowptr + i + 1, pol);
        bi = ld_b(p, i, pol);
    }
    lean_rows<PROTO, UPPER, UNIT>(p, i, act, lean_load<UPPER, UNIT>(p, act, rs, re, pol), bi, epoch, lane, pol);
}

}  // namespace sptrsv_dev
