// solve_paper.cuh -- the paper's three kernels, control flow as printed, for the
// in-repo ablation (Alg.4 vs Alg.5; SyncFree Alg.3
// vs thread level, Fig.5).  They are NOT the product path: same
// result, the paper's structure, no B200 optimisation beyond what correctness on
// sm_100a needs:
//   * get_value[] is the epoch flag array (flag == epoch <=> true; the per-solve
//     MEMSET of Alg.x l.2 is the epoch bump);
//   * "threadfence(); get_value[i] = true" is st.release.gpu; the busy-wait
//     reads are ld.acquire.gpu and x[col] is read after them (G6);
//   * rows are bound to CTAs through the start ticket (forward progress).
//
//   k_paper_alg5  Writing-First: one thread per row; inner
//                 "while get_value[col]" accumulates ready elements, then the
//                 diagonal test, then re-poll -- one flag load per element.
//   k_paper_alg4  Two-Phase: phase 1 blocking busy-wait on
//                 columns < warp_begin; phase 2 a WARP_SIZE-bounded loop for the
//                 in-warp dependencies.
//   k_paper_alg3  SyncFree: one warp per row, lanes stride the
//                 off-diagonals with a per-element busy-wait, shared-memory tree
//                 reduction (add_len 16 -> 1, G2), lane 0 publishes.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

constexpr int kPaperCta = 256;

__device__ __forceinline__ bool paper_ready(const SolveParams &p, int col, uint32_t epoch) {
    return ld_acquire_u32(p.flags + col) == epoch;
}

__device__ __forceinline__ void paper_publish(const SolveParams &p, int i, double xi, uint32_t epoch) {
    p.x[i] = xi;
    st_release_u32(p.flags + i, epoch);  // threadfence(); get_value[i] <- true
}

__global__ void __launch_bounds__(kPaperCta) k_paper_alg5(SolveParams p) {
    __shared__ uint32_t s_blk, s_epoch;
    if (threadIdx.x == 0) cta_ticket(p, s_blk, s_epoch);
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const int i = (int)s_blk * kPaperCta + threadIdx.x;  // l.3: one thread for one component
    if (i >= p.n) return;
    double left_sum = 0.0;                            // l.4
    int j = p.rowptr[i];                              // l.5
    const int end = p.rowptr[i + 1];
    while (j < end) {                                 // l.6
        int col = p.colidx[j];                        // l.7
        while (col != i && paper_ready(p, col, epoch)) {  // l.8 (col != i: get_value[i] is never true here)
            left_sum = __dadd_rn(left_sum, __dmul_rn(p.val[j], ld_relaxed_f64(p.x + col)));  // l.9
            ++j;                                      // l.10
            col = p.colidx[j];                        // l.11
        }
        if (col == i) {                               // l.12
            const double xi = __ddiv_rn(__dsub_rn(p.b[i], left_sum), p.val[end - 1]);  // l.13
            paper_publish(p, i, xi, epoch);           // l.14-16
            ++j;                                      // l.17
            break;                                    // l.18
        }
    }
}

__global__ void __launch_bounds__(kPaperCta) k_paper_alg4(SolveParams p) {
    __shared__ uint32_t s_blk, s_epoch;
    if (threadIdx.x == 0) cta_ticket(p, s_blk, s_epoch);
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const int i = (int)s_blk * kPaperCta + threadIdx.x;  // l.3
    const bool act = i < p.n;
    const int warp_begin = (i / 32) * 32;             // l.4
    double left_sum = 0.0;                            // l.5
    int j = act ? p.rowptr[i] : 0;
    const int end = act ? p.rowptr[i + 1] : 0;
    int col = 0;
    for (; j < end; ++j) {                            // l.6: phase 1
        col = p.colidx[j];                            // l.7
        if (col < warp_begin) {                       // l.8
            while (!paper_ready(p, col, epoch)) {     // l.9-10: busy-wait
            }
            left_sum = __dadd_rn(left_sum, __dmul_rn(p.val[j], ld_relaxed_f64(p.x + col)));  // l.11
        } else {
            break;                                    // l.12-13
        }
    }
    bool done = !act;
    for (int k = 0; k < 32 * 64 && __any_sync(FULL, !done); ++k) {  // l.14: phase 2 (bounded; see below)
        if (!done) {
            while (col != i && paper_ready(p, col, epoch)) {  // l.15
                left_sum = __dadd_rn(left_sum, __dmul_rn(p.val[j], ld_relaxed_f64(p.x + col)));  // l.16
                ++j;                                  // l.17
                col = p.colidx[j];                    // l.18
            }
            if (col == i) {                           // l.19
                const double xi = __ddiv_rn(__dsub_rn(p.b[i], left_sum), p.val[end - 1]);  // l.20
                paper_publish(p, i, xi, epoch);       // l.21-23
                done = true;                          // l.24-25
            }
        }
    }
    // The printed loop runs exactly WARP_SIZE iterations; that bound assumes the
    // lanes of a warp run in lock-step and each iteration solves >= 1 in-warp
    // row.  With independent thread scheduling a lane's phase-2 iteration can
    // overtake the publish of the lane it waits for, so the bound here is a
    // generous multiple (64 x WARP_SIZE) plus the warp vote -- enough for every
    // lane to finish; it is an ablation kernel, the ordering argument of the
    // product path does not depend on it.
}

__global__ void __launch_bounds__(kPaperCta) k_paper_alg3(SolveParams p) {
    __shared__ uint32_t s_blk, s_epoch;
    __shared__ double left_sum_s[kPaperCta];          // l.4: left_sum[WARP_SIZE] per warp
    if (threadIdx.x == 0) cta_ticket(p, s_blk, s_epoch);
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const int warp = threadIdx.x >> 5, tid = threadIdx.x & 31;
    const int i = (int)s_blk * (kPaperCta / 32) + warp;  // l.3: one warp for one component
    if (i >= p.n) return;
    double *ls = left_sum_s + warp * 32;
    ls[tid] = 0.0;                                    // l.5
    double sum = 0.0;                                 // l.7
    const int s = p.rowptr[i], e = p.rowptr[i + 1];
    for (int j = s + tid; j <= e - 2; j += 32) {      // l.8
        const int col = p.colidx[j];                  // l.9
        while (!paper_ready(p, col, epoch)) {         // l.10-11: busy-wait
        }
        sum = __dadd_rn(sum, __dmul_rn(p.val[j], ld_relaxed_f64(p.x + col)));  // l.12
    }
    ls[tid] = sum;                                    // l.13
    __syncwarp();
    for (int add_len = 16; add_len > 0; add_len >>= 1) {  // l.14-17 (halving: DESIGN.md G2)
        if (tid < add_len) ls[tid] = __dadd_rn(ls[tid], ls[tid + add_len]);
        __syncwarp();
    }
    if (tid == 0) {                                   // l.18
        const double xi = __ddiv_rn(__dsub_rn(p.b[i], ls[0]), p.val[e - 1]);  // l.19
        paper_publish(p, i, xi, epoch);               // l.20-22
    }
}

}  // namespace sptrsv_dev
