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

// PLAN_WARP: task t = logical row t.  PLAN_LIST: tasks[t] >= 0 is a 32-row thread-level
// group starting at that logical row (one row per lane, lean_rows), ~row a warp-level row;
// the list is in logical (ticket) order, built by build_plan over reversed rows for UPPER.
template <int PROTO, bool UPPER, bool UNIT, int PLAN>
__global__ void __launch_bounds__(kTriWarpCta) k_solve_tri_warp(SolveParams p) {
    __shared__ uint32_t s_blk, s_epoch;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        cta_ticket(p, s_blk, s_epoch);
        if (p.bflag) {  // sptrsv_solve_host: the b chunks of this CTA's tasks' (physical) rows
            int lo = p.n, hi = 0;  // logical row range of the CTA's tasks
            for (int t = (int)s_blk * (kTriWarpCta / 32); t < min(p.n_tasks, ((int)s_blk + 1) * (kTriWarpCta / 32)); ++t) {
                int r0 = t, r1 = t + 1;
                if (PLAN == PLAN_LIST) {
                    const int v = p.tasks[t];
                    r0 = v >= 0 ? v : ~v;
                    r1 = v >= 0 ? min(p.n, v + 32) : r0 + 1;
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
    const int task = (int)s_blk * (kTriWarpCta / 32) + warp;
    if (task >= p.n_tasks) return;
    const uint64_t pol = policy_evict_first();
    p.local = 0;
    if (PLAN == PLAN_WARP) {
        tri_warp_row<PROTO, UPPER, UNIT>(p, task, epoch, lane, pol);
        return;
    }
    const int t = __ldg(p.tasks + task);
    if (t < 0) {
        tri_warp_row<PROTO, UPPER, UNIT>(p, ~t, epoch, lane, pol);
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
    lean_rows<PROTO, UPPER, UNIT>(p, i, act, rs, re, bi, epoch, lane, pol);
}

}  // namespace sptrsv_dev
