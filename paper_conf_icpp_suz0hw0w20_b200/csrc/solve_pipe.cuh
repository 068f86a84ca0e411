// solve_pipe.cuh -- the pipelined solve engine (ENGINE_PIPE, the default).
//
// Same method as k_solve (Writing-First thread-level rows, Alg.5 PAPER.md:305-325,
// and warp-level long rows, Alg.3, in original row order, no
// level preprocessing), organised for B200:
//
//   * persistent CTAs (grid = resident capacity), each with W compute warps and
//     ONE loader warp (warp specialisation);
//   * work unit = a ROUND = W consecutive warp tasks (a contiguous row range);
//     the loader takes rounds in row order from an atomic ticket -- the same
//     forward-progress argument as the one-shot engine: a round is only held by
//     a running CTA, rounds are processed in ticket order, so the lowest
//     unfinished round is always being worked on;
//   * the loader streams each round's rowptr / b / colidx / val into an S-stage
//     shared-memory ring with 1-D TMA bulk copies (cp.async.bulk, completion
//     counted on an mbarrier) -- the CSR stream never passes through registers,
//     and the DRAM latency of round k+1..k+S-1 overlaps the dependency waits of
//     round k;
//   * compute warps wait on the stage's "full" mbarrier, solve their task from
//     shared memory (dependencies inside the round through the stage's x copy,
//     the rest through the global ready protocol), and release the stage on its
//     "empty" mbarrier.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

// Stage header (first 64 bytes of each stage).
struct StageHdr {
    int q;            // round index; -1 = end of work
    int t0, t1;       // tasks [t0, t1)
    int r0, r1;       // rows [r0, r1)
    int rp_off;       // global element index held by rp[0]
    int b_off;        // ... by b[0]
    int c_off;        // ... by col[0]
    int v_off;        // ... by val[0]
    int staged;       // colidx/val of the round are in the stage (else read from global)
    int pad[6];
};

struct PipeGeom {  // byte offsets inside one stage, and sizes
    int W;         // compute warps per CTA
    int S;         // ring stages
    int RB;        // rows per round, max (32 * W)
    int E;         // colidx/val entries per stage
    int B;         // rounds per ticket
    int off_rp, off_b, off_col, off_val, off_xc, stage_bytes;
};

// Copy elements [lo, hi) of a global array (element size ES, L elements, base
// 16-byte aligned) to shared address sdst (16-byte aligned): the 16-byte aligned
// body by TMA bulk copy, the last < 16 bytes before the array end (only at the
// very end of the array) by plain loads.  Returns the element index stored at
// sdst; adds the bulk bytes to *tx and, if issue, issues the copy (lane 0).
template <int ES>
__device__ __forceinline__ int stage_span(const void *g, long long lo, long long hi, long long L, unsigned sdst,
                                          unsigned *tx, int lane, bool tails, bool issue, unsigned bar,
                                          uint64_t pol) {
    const long long a_lo = (lo * ES) & ~15ll;
    const long long a_hi = ((hi * ES) + 15) & ~15ll;
    const long long lim = (L * ES) & ~15ll;
    long long b_end = a_hi < lim ? a_hi : lim;
    if (b_end < a_lo) b_end = a_lo;
    const unsigned bytes = (hi > lo) ? (unsigned)(b_end - a_lo) : 0u;
    if (tails && hi > lo) {
        // elements past the last full 16-byte block of the array
        for (long long e = b_end / ES + lane; e < hi; e += 32) {
            if (e < lo) continue;
            const unsigned dst = sdst + (unsigned)(e * ES - a_lo);
            if (ES == 4) {
                const int v = ld_stream_i32(reinterpret_cast<const int32_t *>(g) + e, pol);
                asm volatile("st.shared.b32 [%0], %1;" ::"r"(dst), "r"(v) : "memory");
            } else {
                const double v = ld_stream_f64(reinterpret_cast<const double *>(g) + e, pol);
                asm volatile("st.shared.f64 [%0], %1;" ::"r"(dst), "d"(v) : "memory");
            }
        }
    }
    if (tx) *tx += bytes;
    if (issue && bytes)
        bulk_g2s(sdst, reinterpret_cast<const char *>(g) + a_lo, bytes, bar, pol);
    return (int)(a_lo / ES);
}

template <int PLAN>
__device__ __forceinline__ int round_row(const SolveParams &p, int t) {
    if (t >= p.n_tasks) return p.n;
    if (PLAN == PLAN_THREAD) return t * 32;
    if (PLAN == PLAN_WARP) return t;
    return task_row(__ldg(p.tasks + t));
}

// ---------------------------------------------------------------- loader warp
//
// Rounds are taken one ticket at a time (consecutive rounds land in different
// CTAs, so a CTA never queues a round behind its own predecessor) with a deep
// lane-parallel lookahead so that neither the ticket atomic nor the dependent
// rowptr loads of a round are ever waited for:
//   lane k % kLA holds the round consumed at iteration k; right after staging it
//   the lane takes the ticket of the round it will stage kLA iterations later,
//   and kD iterations after that it issues that round's rowptr bounds loads.
// Tickets taken later are larger, and each lane's rounds are staged in ticket
// order, so the CTA stages its rounds in increasing order (forward progress).
constexpr int kLA = 12;
constexpr int kLD = 4;

struct RoundInfo {
    int t0, t1, r0, r1, e0, e1;
    bool valid;
};

template <int PLAN>
__device__ __forceinline__ RoundInfo round_info(const SolveParams &p, const PipeGeom &g, unsigned q, uint64_t pol) {
    RoundInfo ri;
    const long long t0l = (long long)q * g.W;
    ri.valid = t0l < p.n_tasks;
    ri.t0 = ri.valid ? (int)t0l : 0;
    ri.t1 = ri.valid ? min(p.n_tasks, ri.t0 + g.W) : 0;
    ri.r0 = ri.valid ? round_row<PLAN>(p, ri.t0) : 0;
    ri.r1 = ri.valid ? round_row<PLAN>(p, ri.t1) : 0;
    ri.e0 = ri.valid ? ld_stream_i32(p.rowptr + ri.r0, pol) : 0;
    ri.e1 = ri.valid ? ld_stream_i32(p.rowptr + ri.r1, pol) : 0;
    return ri;
}

template <int PLAN>
__device__ void pipe_loader(const SolveParams &p, const PipeGeom &g, unsigned char *ring, unsigned full0,
                            unsigned empty0, int lane, uint64_t pol, uint32_t *wt) {
    const unsigned ring_s = smem_u32(ring);
    unsigned tq = 0;
    RoundInfo ri = {};
    // prologue: tickets for the first kLA rounds (in lane order), then their bounds
    for (int j = 0; j < kLA; ++j) {
        if (lane == j) tq = atomicAdd(wt, 1u);
        __syncwarp();
    }
    if (lane < kLA) ri = round_info<PLAN>(p, g, tq, pol);
    for (int k = 0;; ++k) {
        const int c = k % kLA;
        const int s = k % g.S;
        const unsigned full = full0 + 8u * s, empty = empty0 + 8u * s;
        unsigned char *st = ring + (size_t)s * g.stage_bytes;
        const unsigned st_s = ring_s + (unsigned)s * g.stage_bytes;
        if (k >= g.S) {  // wait until the compute warps released this stage
            const unsigned par = (unsigned)((k / g.S) - 1) & 1u;
            unsigned spins = 0;
            while (!mbar_try_wait(empty, par)) {
                if ((++spins & 1023u) == 0 && ld_relaxed_u32(&p.st->abort.v)) return;
            }
        }
        StageHdr *h = reinterpret_cast<StageHdr *>(st);
        const bool v = __shfl_sync(FULL, ri.valid, c);
        if (!v) {  // end of work: an empty stage with q = -1
            if (lane == 0) {
                h->q = -1;
                mbar_arrive_expect_tx(full, 0);
            }
            return;
        }
        const int R0 = __shfl_sync(FULL, ri.r0, c), R1 = __shfl_sync(FULL, ri.r1, c);
        const int T0 = __shfl_sync(FULL, ri.t0, c), T1 = __shfl_sync(FULL, ri.t1, c);
        const int E0 = __shfl_sync(FULL, ri.e0, c), E1 = __shfl_sync(FULL, ri.e1, c);
        const unsigned Q = __shfl_sync(FULL, tq, c);
        // lookahead upkeep: lane c takes the ticket of its next round; the lane that took a
        // ticket kLD iterations ago issues that round's bounds loads
        if (lane == c) tq = atomicAdd(wt, 1u);
        if (k >= kLD && lane == (k - kLD) % kLA) ri = round_info<PLAN>(p, g, tq, pol);
        const bool staged = (E1 - E0) <= g.E;
        // x copy of the round := sentinel (dependencies inside the round poll it)
        unsigned long long *xc = reinterpret_cast<unsigned long long *>(st + g.off_xc);
        for (int r = lane; r < R1 - R0; r += 32) xc[r] = kSentinel;
        unsigned tx = 0;
        // tails first (plain stores), then one arrive.expect_tx, then the bulk copies
        const long long nnz = p.nnz;
        const int rp_off = stage_span<4>(p.rowptr, R0, R1 + 1, (long long)p.n + 1, st_s + g.off_rp, &tx, lane,
                                         true, false, full, pol);
        const int b_off = stage_span<8>(p.b, R0, R1, p.n, st_s + g.off_b, &tx, lane, true, false, full, pol);
        int c_off = 0, v_off = 0;
        if (staged) {
            c_off = stage_span<4>(p.colidx, E0, E1, nnz, st_s + g.off_col, &tx, lane, true, false, full, pol);
            v_off = stage_span<8>(p.val, E0, E1, nnz, st_s + g.off_val, &tx, lane, true, false, full, pol);
        }
        if (lane == 0) {
            h->q = (int)Q;
            h->t0 = T0;
            h->t1 = T1;
            h->r0 = R0;
            h->r1 = R1;
            h->rp_off = rp_off;
            h->b_off = b_off;
            h->c_off = c_off;
            h->v_off = v_off;
            h->staged = staged;
        }
        __syncwarp();
        if (lane == 0) {
            mbar_arrive_expect_tx(full, tx);
            stage_span<4>(p.rowptr, R0, R1 + 1, (long long)p.n + 1, st_s + g.off_rp, nullptr, 0, false, true,
                          full, pol);
            stage_span<8>(p.b, R0, R1, p.n, st_s + g.off_b, nullptr, 0, false, true, full, pol);
            if (staged) {
                stage_span<4>(p.colidx, E0, E1, nnz, st_s + g.off_col, nullptr, 0, false, true, full, pol);
                stage_span<8>(p.val, E0, E1, nnz, st_s + g.off_val, nullptr, 0, false, true, full, pol);
            }
        }
        __syncwarp();
    }
}

// ---------------------------------------------------------------- compute warp
template <int PLAN, int PROTO>
__device__ bool pipe_compute(const SolveParams &p, const PipeGeom &g, unsigned char *ring, unsigned full0,
                             unsigned empty0, int warp, int lane, uint32_t epoch, uint64_t pol) {
    const unsigned ring_s = smem_u32(ring);
    for (int k = 0;; ++k) {
        const int s = k % g.S;
        const unsigned full = full0 + 8u * s, empty = empty0 + 8u * s;
        const unsigned char *st = ring + (size_t)s * g.stage_bytes;
        {
            const unsigned par = (unsigned)(k / g.S) & 1u;
            unsigned spins = 0;
            while (!mbar_try_wait(full, par)) {
                if ((++spins & 1023u) == 0 && ld_relaxed_u32(&p.st->abort.v)) return false;
            }
        }
        const StageHdr *h = reinterpret_cast<const StageHdr *>(st);
        if (h->q < 0) return true;
        const int t = h->t0 + warp;
        bool ok = true;
        if (t < h->t1) {
            const int32_t *rp = reinterpret_cast<const int32_t *>(st + g.off_rp) - h->rp_off;
            const double *bb = reinterpret_cast<const double *>(st + g.off_b) - h->b_off;
            // one code path: generic pointers to the staged slice, or to global memory
            const int32_t *cp = h->staged ? reinterpret_cast<const int32_t *>(st + g.off_col) - h->c_off : p.colidx;
            const double *vp = h->staged ? reinterpret_cast<const double *>(st + g.off_val) - h->v_off : p.val;
            Cta cta;
            cta.xc = reinterpret_cast<unsigned long long *>(const_cast<unsigned char *>(st) + g.off_xc);
            cta.xc_s = ring_s + (unsigned)s * g.stage_bytes + g.off_xc;
            cta.R0 = h->r0;
            cta.R1 = h->r1;
            int tv = t;
            if (PLAN == PLAN_LIST) tv = __ldg(p.tasks + t);
            const bool thread_level = (PLAN == PLAN_THREAD) || (PLAN == PLAN_LIST && tv >= 0);
            auto col_at = [&](int jj) -> int { return cp[jj]; };
            auto val_at = [&](int jj) -> double { return vp[jj]; };
            if (thread_level) {
                const int r0 = (PLAN == PLAN_THREAD) ? t * 32 : tv;
                const int rows = min(32, p.n - r0);
                const bool act = lane < rows;
                const int i = r0 + lane;
                const int rs = act ? rp[i] : 0;
                const int re = act ? rp[i + 1] : 1;
                const double bi = act ? bb[i] : 0.0;
                ok = thread_rows<PROTO>(p, cta, i, act, rs, re, bi, epoch, lane, col_at, val_at);
            } else {
                const int i = (PLAN == PLAN_WARP) ? t : ~tv;
                const int rs = rp[i], re = rp[i + 1];
                ok = warp_row<PROTO>(p, cta, i, rs, re, bb[i], vp[re - 1], epoch, lane, col_at, val_at);
            }
        }
        __syncwarp();
        if (!ok) return false;
        if (lane == 0) mbar_arrive(empty);
    }
}

template <int PLAN, int PROTO>
__global__ void __launch_bounds__(1024) k_solve_pipe(SolveParams p, PipeGeom g) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ __align__(8) unsigned long long bars[2 * 8];  // full[S], empty[S] (S <= 8)
    __shared__ uint32_t s_epoch, s_blk;
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const unsigned full0 = smem_u32(&bars[0]), empty0 = smem_u32(&bars[8]);
    if (threadIdx.x == 0) {
        for (int s = 0; s < g.S; ++s) {
            mbar_init(full0 + 8u * s, 1);
            mbar_init(empty0 + 8u * s, (unsigned)g.W);
        }
        fence_mbar_init();
        cta_ticket(p, s_blk, s_epoch);
        p.st->wtick[(s_epoch + 1u) & 1u].v = 0;  // the next solve's work counter
    }
    __syncthreads();
    const uint32_t epoch = s_epoch;
    const uint64_t pol = policy_evict_first();
    if (warp == g.W)
        pipe_loader<PLAN>(p, g, smem, full0, empty0, lane, pol, &p.st->wtick[epoch & 1u].v);
    else
        pipe_compute<PLAN, PROTO>(p, g, smem, full0, empty0, warp, lane, epoch, pol);
}

}  // namespace sptrsv_dev
