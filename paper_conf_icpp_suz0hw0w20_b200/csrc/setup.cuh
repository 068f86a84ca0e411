// setup.cuh -- O(nnz) analyse kernels (SURVEY/DESIGN row a1).
//
//   k_validate   per-row CSR checks (the shape Alg.1 assumes: PAPER.md:72,
//                :89-91), in-degree, longest row
//   k_plan_count per 32-row group: thread- or warp-level (sec.4.4,
//                PAPER.md:329-335) -> tasks per group, block totals
//   k_plan_write block-local exclusive scan + host-scanned block offsets ->
//                the row-ordered task list
// None of this is level analysis: it reads each row once, in row order.
#pragma once
#include <cstdint>

namespace sptrsv_dev {

enum : int {  // same numbering as sptrsv_status (negated)
    E_INVALID_ARG = 1, E_NOT_LOWER = 2, E_MISSING_DIAG = 3, E_ZERO_DIAG = 4, E_UNSORTED = 5, E_BAD_ROWPTR = 6,
    E_BAD_COL = 7
};

// Everything analyse learns on the device, read back by the host in ONE copy at the end
// (sptrsv.cu sptrsv_analyse_csr_ex): the whole setup is a handful of kernels on one stream.
struct AnalyseOut {
    unsigned long long status;   // min over ((row + 1) << 8 | code); key 0 << 8 | code: a global
                                 // rowptr error; ~0 = valid (the lowest offending row wins)
    long long nnz;               // rowptr[n]
    int32_t max_row;             // longest row (entries)
    int32_t threshold;           // AUTO warp threshold the plan used (sec.4.4)
    int32_t med_log2;            // floor(log2(median nearest-dependency distance)), -1 = none
    int32_t n_tasks, n_tgroups;  // plan: warp tasks, 32-row thread groups
    int32_t n_subtasks;          // plan: tasks with 2..16 lanes per row (sub-warp rows)
    int32_t epl;                 // sub-warp target off-diagonals per lane (0: warp rows only)
    int32_t mid_breaks;          // rows not at a 64-row boundary (logical order) without a previous-row
                                 // dependency: where CHAIN's in-warp order would serialise independent runs
    unsigned long long near;     // near_deps | warp_deps << 32
    unsigned long long prev;     // prev_deps | near_rows << 32
    unsigned long long hist[32]; // rows by floor(log2(nearest-dependency distance))
    // ENGINE_GRID eligibility (solve_grid.cuh k_grid_probe / k_grid_check): the line length m the
    // probe proposes (0 = none), and over every row for that m: rows violating the band order,
    // north / west entries (register / shuffle operands), far entries (polled)
    int32_t grid_m;
    int32_t grid_viol;
    long long grid_fast;
    long long grid_far;
};

// status: 64-bit min over (row << 8 | code) -> the lowest offending row wins,
// which is the row-ordered error the oracle reports too.
// Also counts "near" dependencies (|i - col| < 256: produced within about one CTA
// of rows) and in-warp ones (i and col in the same 32-row group) -- the statistics
// ENGINE_AUTO uses to choose between the LEAN, ONE-SHOT and CHAIN engines.
// tri: bit 0 UPPER (entries j >= i, diagonal FIRST), bit 1 UNIT
// (diagonal implicit 1, not stored: entries strictly inside the triangle).
__global__ void __launch_bounds__(256) k_validate(const int32_t *__restrict__ rowptr,
                                                  const int32_t *__restrict__ colidx,
                                                  const double *__restrict__ val, int32_t n,
                                                  int32_t *indeg, AnalyseOut *out, int tri) {
    const bool upper = tri & 1, unit = tri & 2;
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    unsigned long long *status = &out->status;
    int32_t *max_row = &out->max_row;
    unsigned long long *near_deps = &out->near;  // near, prev, hist[32] are consecutive
    const int64_t nnz = rowptr[n];  // the nnz the caller's rowptr declares
    if (i == 0) {
        out->nnz = nnz;
        if (rowptr[0] != 0 || nnz < 0) atomicMin(status, (unsigned long long)E_BAD_ROWPTR);  // key row 0: global
        // a row with entries needs colidx / val (unit handles may pass NULL for an empty matrix)
        if (nnz > 0 && (!colidx || (!val && !unit))) atomicMin(status, (unsigned long long)E_INVALID_ARG);
    }
    if (nnz > 0 && (!colidx || (!val && !unit))) return;
    int len = 0;
    unsigned near = 0, wdep = 0, pdep = 0, nrow = 0, mbrk = 0;
    int dmin = 0x7fffffff;  // the row's nearest dependency (distance in rows)
    if (i < n) {
        const int64_t s = rowptr[i], e = rowptr[i + 1];
        int code = 0;
        if (s < 0 || e < s || e > nnz) {
            code = E_BAD_ROWPTR;
        } else if (e == s && !unit) {
            code = E_MISSING_DIAG;
        } else {
            int prev = -1;
            for (int64_t j = s; j < e; ++j) {
                const int c = colidx[j];
                if (c < 0) { code = E_BAD_COL; break; }
                // outside the triangle (for UNIT the diagonal itself is outside too)
                if (upper ? (c < i || (unit && c == i)) : (c > i || (unit && c == i))) { code = E_NOT_LOWER; break; }
                if (c >= n) { code = E_BAD_COL; break; }  // upper only (lower has c <= i < n)
                if (j > s && c <= prev) { code = E_UNSORTED; break; }
                if (c != i && (c > i ? c - i : i - c) < 256) ++near;
                // same 32-row group of LOGICAL rows (upper handles run row n-1-r as logical r)
                if (c != i && (upper ? ((n - 1 - c) >> 5) == ((n - 1 - i) >> 5) : (c >> 5) == (i >> 5))) ++wdep;
                if (c == (upper ? i + 1 : i - 1)) ++pdep;  // the previous row in solve order (chains)
                if (c != i) dmin = min(dmin, c > i ? c - i : i - c);
                prev = c;
            }
            if (!code && !unit) {
                const int64_t jd = upper ? s : e - 1;  // diagonal: first (upper) / last (lower)
                if (colidx[jd] != i) code = E_MISSING_DIAG;
                else if (val[jd] == 0.0) code = E_ZERO_DIAG;
            }
        }
        if (!code && dmin < 256) nrow = 1;  // the row's latest-solved dependency is near
        if (!code && pdep == 0 && ((upper ? n - 1 - i : i) & 63) != 0) mbrk = 1;
        if (!code && dmin != 0x7fffffff) {  // histogram of floor(log2(nearest-dependency distance))
            const int bk = 31 - __clz(dmin);
            const unsigned same = __match_any_sync(__activemask(), bk);
            if ((threadIdx.x & 31) == __ffs(same) - 1)
                atomicAdd(near_deps + 2 + bk, (unsigned long long)__popc(same));
        }
        if (code) atomicMin(status, ((unsigned long long)(i + 1) << 8) | (unsigned long long)code);
        len = code ? 0 : (int)(e - s);
        indeg[i] = code ? 0 : (int)(e - s - (unit ? 0 : 1));
    }
    for (int off = 16; off > 0; off >>= 1) {
        len = max(len, __shfl_xor_sync(0xffffffffu, len, off));
        near += __shfl_xor_sync(0xffffffffu, near, off);
        wdep += __shfl_xor_sync(0xffffffffu, wdep, off);
        pdep += __shfl_xor_sync(0xffffffffu, pdep, off);
        nrow += __shfl_xor_sync(0xffffffffu, nrow, off);
        mbrk += __shfl_xor_sync(0xffffffffu, mbrk, off);
    }
    if ((threadIdx.x & 31) == 0 && mbrk) atomicAdd(&out->mid_breaks, (int)mbrk);
    if ((threadIdx.x & 31) == 0 && len > 0) atomicMax(max_row, len);
    // both totals are < nnz < 2^31: near in the low word, wdep in the high word
    if ((threadIdx.x & 31) == 0 && (near | wdep))
        atomicAdd(near_deps, (unsigned long long)near | ((unsigned long long)wdep << 32));
    // previous-row dependencies in the low word, rows with a near (< 256) nearest dependency in the high word
    if ((threadIdx.x & 31) == 0 && (pdep | nrow))
        atomicAdd(near_deps + 1, (unsigned long long)pdep | ((unsigned long long)nrow << 32));
}

// mode: 0 auto, 1 all thread-level, 2 all warp-level, 3 all sub-warp (width from the group's mean).
// A group of `rows` rows goes beyond thread level in auto mode when its nnz (diagonals
// included) exceeds threshold * rows, i.e. mean nnz/row > threshold (sec.4.4).
// Its width W (lanes per row) is then 32 (a warp per row, Alg.3), or -- with sub-warp rows enabled
// (epl = target off-diagonals per lane) -- the smallest power of two in [2, 32] with
// W * epl >= mean off-diagonals per row: 32 / W rows share one warp task.
// rev (f4 UPPER): groups are over LOGICAL rows r -> row n-1-r (the solve order).
// Returns the group's tasks; *width = 0 (thread level: one task), 32 (one task per row) or W.
__device__ __forceinline__ int group_tasks(const int32_t *rowptr, int32_t n, int g, int mode,
                                           int threshold, int epl, int *width, bool rev) {
    const int r0 = g * 32;
    const int rows = min(32, n - r0);
    const long long gnnz = rev ? (long long)rowptr[n - r0] - rowptr[n - r0 - rows]
                               : (long long)rowptr[r0 + rows] - rowptr[r0];
    const bool beyond = (mode >= 2) || (mode == 0 && gnnz > (long long)threshold * rows);
    if (!beyond) {
        *width = 0;
        return 1;
    }
    int w = 32;
    if (mode == 3 || (mode == 0 && epl > 0)) {
        const long long off = gnnz - rows;  // off-diagonals in the group (approx. for unit forms)
        const int e = max(1, epl > 0 ? epl : 4);
        const int wmax = mode == 3 ? 32 : 16;  // AUTO keeps sub-warp rows at <= 16 lanes
        w = 2;
        while (w < wmax && (long long)w * e * rows < off) w <<= 1;
    }
    *width = w;
    const int per = 32 / w;  // rows per task
    return (rows + per - 1) / per;
}

__device__ __forceinline__ int block_exclusive_scan(int v, int *s_warp, int *total) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int inc = v;
    for (int off = 1; off < 32; off <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, inc, off);
        if (lane >= off) inc += t;
    }
    if (lane == 31) s_warp[warp] = inc;
    __syncthreads();
    if (warp == 0) {
        const int nw = blockDim.x >> 5;
        int w = lane < nw ? s_warp[lane] : 0;
        int wi = w;
        for (int off = 1; off < 32; off <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, wi, off);
            if (lane >= off) wi += t;
        }
        if (lane < nw) s_warp[lane] = wi - w;
        if (lane == nw - 1) s_warp[32] = wi;
    }
    __syncthreads();
    *total = s_warp[32];
    const int r = s_warp[warp] + inc - v;
    __syncthreads();
    return r;
}

__global__ void __launch_bounds__(1024) k_plan_count(const int32_t *__restrict__ rowptr, int32_t n,
                                                     int32_t ngroups, int mode, const AnalyseOut *out,
                                                     int32_t *blk_tasks, int32_t *blk_tgroups, bool rev) {
    __shared__ int s_warp[33];
    const int threshold = out->threshold, epl = out->epl;
    const int g = blockIdx.x * blockDim.x + threadIdx.x;
    int t = 0, tg = 0, ts = 0;
    if (g < ngroups) {
        int w;
        t = group_tasks(rowptr, n, g, mode, threshold, epl, &w, rev);
        tg = w == 0 ? 1 : 0;
        ts = (w > 0 && w < 32) ? t : 0;
    }
    int tot_t, tot_g, tot_s;
    block_exclusive_scan(t, s_warp, &tot_t);
    block_exclusive_scan(tg, s_warp, &tot_g);
    block_exclusive_scan(ts, s_warp, &tot_s);
    if (threadIdx.x == 0) {
        blk_tasks[blockIdx.x] = tot_t;
        blk_tgroups[blockIdx.x] = tot_g;
        if (tot_s) atomicAdd(&((AnalyseOut *)out)->n_subtasks, tot_s);  // zeroed by k_auto_threshold
    }
}

__global__ void __launch_bounds__(1024) k_plan_write(const int32_t *__restrict__ rowptr, int32_t n,
                                                     int32_t ngroups, int mode, const AnalyseOut *out,
                                                     const int32_t *__restrict__ blk_offset,
                                                     int32_t *tasks, uint8_t *task_w, bool rev) {
    __shared__ int s_warp[33];
    const int threshold = out->threshold, epl = out->epl;
    const int g = blockIdx.x * blockDim.x + threadIdx.x;
    int t = 0, w = 0;
    if (g < ngroups) t = group_tasks(rowptr, n, g, mode, threshold, epl, &w, rev);
    int tot;
    const int off = block_exclusive_scan(t, s_warp, &tot) + blk_offset[blockIdx.x];
    if (g < ngroups) {
        if (w == 0) {
            tasks[off] = g * 32;  // thread task: the group's first (logical) row
            task_w[off] = 0;
        } else {
            const int per = 32 / w;  // w = 32: one warp task per row (Alg.3); else 32/w rows per task
            for (int k = 0; k < t; ++k) {
                tasks[off + k] = ~(g * 32 + k * per);
                task_w[off + k] = (uint8_t)w;
            }
        }
    }
}

// AUTO's per-32-row-group dispatch (sec.4.4, PAPER.md:329-335 leaves it as future work; SURVEY
// f2): from floor(log2) of the median distance to a row's nearest dependency -- on leveled matrices
// about the level width, which moves the crossover -- the mean nnz/row above which a group leaves
// thread level (threshold) and how many lanes its rows get (epl: target off-diagonals per lane,
// W = smallest power of two with W * epl >= mean off-diagonals, capped at 16; 0 = a warp per row).
// Measured on B200 (profiles/r02_f2_sweep.md, n = 2e5 leveled synthetics + c2 / c4 / c5):
//   < 64 rows            thread level only (in-CTA / in-warp resolution wins)
//   64 .. 511            threshold 2, warp rows (Alg.3)
//   512 .. 1023          threshold 2, sub-warp rows, epl 4   (c4: 16 lanes per 64-entry row)
//   1024 .. 8191         threshold 2, sub-warp rows, epl 2
//   8192 .. 65535        threshold 3, sub-warp rows, epl 8
//   >= 65536             threshold 7, sub-warp rows, epl 8   (c2 / c5 at 2.8 nnz/row stay thread; at
//                        n = 1e6 with 10 levels the persistent thread engine LEANP beats sub-warp rows
//                        up to ~7 nnz/row: 4 nnz/row 41 vs 72 us, 6 nnz/row 56 vs 72 us --
//                        profiles/r02_auto/lev_1m_sweep.txt)
//   n <= 1024            thread level only (one 1024-thread one-shot CTA resolves it in smem)
// user >= 0 / user_epl >= 0: SPTRSV_OPT_WARP_THRESHOLD / SPTRSV_OPT_SUBWARP were set.  One thread.
__global__ void k_auto_threshold(AnalyseOut *out, int32_t n, int32_t user, int32_t user_epl) {
    out->n_subtasks = 0;
    unsigned long long tot = 0, acc = 0;
    for (int k = 0; k < 32; ++k) tot += out->hist[k];
    int med = -1;
    for (int k = 0; k < 32 && tot; ++k) {
        acc += out->hist[k];
        if (2 * acc >= tot) {
            med = k;
            break;
        }
    }
    out->med_log2 = med;
    int t, e;
    if (n <= 1024) t = 1 << 30, e = 0;
    else if (med < 0) t = 16, e = 0;  // no dependencies at all
    else if (med <= 5) t = 1 << 30, e = 0;
    else if (med <= 8) t = 2, e = 0;
    else if (med <= 9) t = 2, e = 4;
    else if (med <= 12) t = 2, e = 2;
    else if (med <= 15) t = 3, e = 8;
    else t = 7, e = 8;  // >= 65536 rows: very wide levels, thread rows (LEANP) win up to ~7 nnz/row
    out->threshold = user >= 0 ? user : t;
    out->epl = user_epl >= 0 ? user_epl : e;
}

// exclusive scan of the per-block task / thread-group counts (one CTA, any number of blocks):
// blk_offset[b] = tasks before block b; out->n_tasks / n_tgroups = the totals
__global__ void __launch_bounds__(1024) k_plan_scan(const int32_t *__restrict__ blk_tasks,
                                                    const int32_t *__restrict__ blk_tgroups, int32_t nb,
                                                    int32_t *blk_offset, AnalyseOut *out) {
    __shared__ int s_warp[33];
    long long carry = 0, carry_g = 0;
    for (int b0 = 0; b0 < nb; b0 += blockDim.x) {
        const int b = b0 + threadIdx.x;
        const int v = b < nb ? blk_tasks[b] : 0;
        const int g = b < nb ? blk_tgroups[b] : 0;
        int tot, totg;
        const int ex = block_exclusive_scan(v, s_warp, &tot);
        block_exclusive_scan(g, s_warp, &totg);
        if (b < nb) blk_offset[b] = (int32_t)(carry + ex);
        carry += tot;
        carry_g += totg;
    }
    if (threadIdx.x == 0) {
        out->n_tasks = (int32_t)carry;
        out->n_tgroups = (int32_t)carry_g;
    }
}

}  // namespace sptrsv_dev
