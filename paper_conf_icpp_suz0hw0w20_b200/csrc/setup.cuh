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
    int32_t pad;
    unsigned long long near;     // near_deps | warp_deps << 32
    unsigned long long prev;     // prev_deps | near_rows << 32
    unsigned long long hist[32]; // rows by floor(log2(nearest-dependency distance))
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
    unsigned near = 0, wdep = 0, pdep = 0, nrow = 0;
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
    }
    if ((threadIdx.x & 31) == 0 && len > 0) atomicMax(max_row, len);
    // both totals are < nnz < 2^31: near in the low word, wdep in the high word
    if ((threadIdx.x & 31) == 0 && (near | wdep))
        atomicAdd(near_deps, (unsigned long long)near | ((unsigned long long)wdep << 32));
    // previous-row dependencies in the low word, rows with a near (< 256) nearest dependency in the high word
    if ((threadIdx.x & 31) == 0 && (pdep | nrow))
        atomicAdd(near_deps + 1, (unsigned long long)pdep | ((unsigned long long)nrow << 32));
}

// mode: 0 auto, 1 all thread-level, 2 all warp-level.
// A group of `rows` rows goes warp-level in auto mode when its nnz (diagonals
// included) exceeds threshold * rows, i.e. mean nnz/row > threshold.
// rev (f4 UPPER): groups are over LOGICAL rows r -> row n-1-r (the solve order).
__device__ __forceinline__ int group_tasks(const int32_t *rowptr, int32_t n, int g, int mode,
                                           int threshold, bool *is_warp, bool rev) {
    const int r0 = g * 32;
    const int rows = min(32, n - r0);
    const long long gnnz = rev ? (long long)rowptr[n - r0] - rowptr[n - r0 - rows]
                               : (long long)rowptr[r0 + rows] - rowptr[r0];
    const bool w = (mode == 2) || (mode == 0 && gnnz > (long long)threshold * rows);
    *is_warp = w;
    return w ? rows : 1;
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
    const int threshold = out->threshold;
    const int g = blockIdx.x * blockDim.x + threadIdx.x;
    int t = 0, tg = 0;
    if (g < ngroups) {
        bool w;
        t = group_tasks(rowptr, n, g, mode, threshold, &w, rev);
        tg = w ? 0 : 1;
    }
    int tot_t, tot_g;
    block_exclusive_scan(t, s_warp, &tot_t);
    block_exclusive_scan(tg, s_warp, &tot_g);
    if (threadIdx.x == 0) {
        blk_tasks[blockIdx.x] = tot_t;
        blk_tgroups[blockIdx.x] = tot_g;
    }
}

__global__ void __launch_bounds__(1024) k_plan_write(const int32_t *__restrict__ rowptr, int32_t n,
                                                     int32_t ngroups, int mode, const AnalyseOut *out,
                                                     const int32_t *__restrict__ blk_offset,
                                                     int32_t *tasks, bool rev) {
    __shared__ int s_warp[33];
    const int threshold = out->threshold;
    const int g = blockIdx.x * blockDim.x + threadIdx.x;
    int t = 0;
    bool w = false;
    if (g < ngroups) t = group_tasks(rowptr, n, g, mode, threshold, &w, rev);
    int tot;
    const int off = block_exclusive_scan(t, s_warp, &tot) + blk_offset[blockIdx.x];
    if (g < ngroups) {
        if (w) {
            for (int k = 0; k < t; ++k) tasks[off + k] = ~(g * 32 + k);  // warp task: row
        } else {
            tasks[off] = g * 32;  // thread task: first row of the group
        }
    }
}

// AUTO's per-32-row-group warp threshold (mean nnz/row above which a group runs warp-level), from
// floor(log2) of the median distance to a row's nearest dependency -- on leveled matrices about the
// level width, which moves the thread/warp crossover (f2 sweep): < 64 rows:
// thread level only; 64..1023: warp from 2 nnz/row; 1024..8191: from 6; wider: from 20.  A system
// that fits one 1024-thread one-shot CTA resolves in shared memory: thread level only.
// user >= 0: SPTRSV_OPT_WARP_THRESHOLD was set, use it.  One thread.
__global__ void k_auto_threshold(AnalyseOut *out, int32_t n, int32_t user) {
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
    int t;
    if (user >= 0) t = user;
    else if (n <= 1024) t = 1 << 30;
    else if (med < 0) t = 16;  // no dependencies at all
    else if (med <= 5) t = 1 << 30;
    else if (med <= 9) t = 2;
    else if (med <= 12) t = 6;
    else t = 20;
    out->threshold = t;
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
