// solve_dyn.cuh -- the dynamic-lane engine (ENGINE_DYN) for all-thread-level plans.
//
// Same per-row method as the other engines (Writing-First, Alg.5 PAPER.md:305-325:
// poll the next dependency, consume in row order with separately rounded
// mul/add, solve + publish at the diagonal).  What changes is WHEN a thread
// takes a row.  The paper binds rows to threads once, at warp start ("we
// distribute tasks at the beginning of the warp execution"), so a
// warp -- and its CTA -- holds its slot until its slowest row finishes; with
// random dependencies that is the end of the previous level, and the in-order
// residency window then advances one level per fill/drain (measured on c2: 84%
// of rows START after their dependency was already published).  Here every lane
// owns K row SLOTS; a slot that publishes takes the next row at once:
//
//   * persistent CTAs; each warp takes CHUNKS of 128 consecutive rows from an
//     atomic ticket (in row order -- the forward-progress argument is the
//     ticket's: rows are dispensed in order, a dispensed row sits in a slot or in
//     its warp's chunk behind only earlier rows, so the lowest unfinished row is
//     always in a slot and its dependencies are done);
//   * the chunk's rowptr[] and b[] are prefetched into shared memory with
//     cp.async one chunk ahead (the ticket two chunks ahead), so a slot's refill
//     costs shared-memory reads;
//   * per slot: FREE -> LOAD (entries and L_ii in flight) -> ACTIVE (one global
//     poll per pass, next entry prefetched) -> publish -> FREE.
// No smem x copy: every dependency goes through the global protocol.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

constexpr int kDynSub = 32;                 // rows per warp sub-chunk (one per lane)
constexpr int kDynCtaChunk = 1024;          // rows per CTA ticket
constexpr int kDynBuf = 4 * 36 + 8 * kDynSub;  // rowptr[33] (padded) + b[32]
constexpr int kDynWarpSmem = 2 * kDynBuf;      // double buffer per warp

__device__ __forceinline__ void cp_async4(unsigned dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async8(unsigned dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// CTA-level dispenser: 1024-row chunks from the global ticket, 32-row sub-chunks
// to the CTA's warps in order under a shared-memory lock.  Returns the first row
// of the warp's next sub-chunk, or >= n when the work is exhausted (lane 0 only).
struct DynPool {
    int base;   // first row of the CTA's current chunk
    int pos;    // next sub-chunk offset in it
    int lock;
};

__device__ __forceinline__ int dyn_next_sub(const SolveParams &p, DynPool *pool, uint32_t *wt) {
    while (atomicCAS(&pool->lock, 0, 1) != 0) nanosleep_ns(32);
    __threadfence_block();
    int r;
    if (pool->pos >= kDynCtaChunk) {
        const unsigned q = atomicAdd(wt, 1u);
        pool->base = (long long)q * kDynCtaChunk < p.n ? (int)(q * kDynCtaChunk) : p.n;
        pool->pos = 0;
    }
    r = pool->base + pool->pos;
    pool->pos += kDynSub;
    if (pool->base >= p.n) r = p.n;
    __threadfence_block();
    atomicExch(&pool->lock, 0);
    return r;
}

// STATIC (template flag): no ticket at all -- warp g of the G*W persistent warps
// takes the 32-row units g, g + G*W, g + 2*G*W, ...  This order is only safe
// when all CTAs are co-resident, so the host launches it cooperatively.
template <int PROTO, int K, bool STATIC>
__global__ void __launch_bounds__(256) k_solve_dyn(SolveParams p) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint32_t s_epoch, s_blk;
    __shared__ DynPool s_pool;
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        cta_ticket(p, s_blk, s_epoch);
        p.st->wtick[(s_epoch + 1u) & 1u].v = 0;  // the next solve's work counter
        s_pool.base = 0;
        s_pool.pos = kDynCtaChunk;  // forces a ticket on first use
        s_pool.lock = 0;
    }
    __syncthreads();
    const uint32_t epoch = s_epoch;
    const uint64_t pol = policy_evict_first();
    unsigned char *wsm = smem + (size_t)warp * kDynWarpSmem;
    auto buf_rp = [&](int c) { return reinterpret_cast<int32_t *>(wsm + c * kDynBuf); };
    auto buf_b = [&](int c) { return reinterpret_cast<double *>(wsm + c * kDynBuf + 4 * 36); };
    // issue the cp.async loads of the sub-chunk starting at row r0 into buffer c (no wait)
    auto load_sub = [&](int r0, int c) {
        if (r0 < p.n) {
            const int rows = min(kDynSub, p.n - r0);
            const unsigned rp_s = smem_u32(buf_rp(c)), b_s = smem_u32(buf_b(c));
            cp_async4(rp_s + 4u * lane, p.rowptr + r0 + min(lane, rows));  // lanes > rows re-read rowptr[r0+rows]
            if (lane == 0) cp_async4(rp_s + 4u * 32, p.rowptr + r0 + rows);
            if (lane < rows) cp_async8(b_s + 8u * lane, p.b + r0 + lane);
        }
        cp_async_commit();
    };
    const long long gwarps = (long long)gridDim.x * (blockDim.x >> 5);
    long long unit = (long long)blockIdx.x * (blockDim.x >> 5) + warp;  // STATIC: this warp's next unit
    auto next_sub = [&]() {
        if (STATIC) {
            const long long r = unit * kDynSub;
            unit += gwarps;
            return r < p.n ? (int)r : p.n;
        }
        int r = 0;
        if (lane == 0) r = dyn_next_sub(p, &s_pool, &p.st->wtick[epoch & 1u].v);
        return __shfl_sync(FULL, r, 0);
    };
    // ---- sub-chunk pipeline: cur (being assigned to slots) and next (loading)
    int s_cur = next_sub();
    int cb = 0;
    load_sub(s_cur, 0);
    int s_nxt = next_sub();
    cp_async_wait_all();
    __syncwarp();
    load_sub(s_nxt, 1);
    int nxt = 0;  // next unassigned row within s_cur
    // ---- slots
    int ri[K], jd[K], j[K], nc[K], nc2[K];
    double nv[K], nv2[K], ls[K], bi[K], dd[K], rr[K];
    unsigned st_load = 0, st_act = 0;  // per-slot bits
#pragma unroll
    for (int k = 0; k < K; ++k) ri[k] = -1;
    uint32_t backoff = p.backoff_min, idle = 0;
    Cta nocta;  // no in-CTA x copy in this engine
    nocta.R0 = nocta.R1 = 0;
    nocta.xc = nullptr;
    nocta.xc_s = 0;
    SolveParams pp = p;
    pp.local = 0;
    while (true) {
        bool prog = false;
        // ---- slots refilled in the previous pass become ACTIVE (their loads had a pass to land)
#pragma unroll
        for (int k = 0; k < K; ++k) {
            if (st_load >> k & 1u) {
                Diag dg;
                dg.init(dd[k]);
                rr[k] = dg.r;
                if (p.trace) p.trace[2 * (size_t)p.n + ri[k]] = globaltimer_ns();
            }
        }
        st_act |= st_load;
        st_load = 0;
        // ---- refill FREE slots with the next rows of the current sub-chunk (in order)
#pragma unroll
        for (int k = 0; k < K; ++k) {
            while (true) {
                const bool free_k = ri[k] < 0;
                const unsigned fm = __ballot_sync(FULL, free_k);
                if (!fm || s_cur >= p.n) break;
                const int rows_cur = min(kDynSub, p.n - s_cur);
                const int avail = rows_cur - nxt;
                const int rank = __popc(fm & ((1u << lane) - 1u));
                if (free_k && rank < avail) {
                    const int idx = nxt + rank;
                    const int32_t *rp = buf_rp(cb);
                    const int rs = rp[idx], re = rp[idx + 1];
                    ri[k] = s_cur + idx;
                    bi[k] = buf_b(cb)[idx];
                    jd[k] = re - 1;
                    j[k] = rs;
                    // entries and the diagonal: in flight until the slot's next pass
                    dd[k] = ld_stream_f64(p.val + jd[k], pol);
                    nc[k] = rs < jd[k] ? ld_stream_i32(p.colidx + rs, pol) : -1;
                    nv[k] = rs < jd[k] ? ld_stream_f64(p.val + rs, pol) : 0.0;
                    nc2[k] = rs + 1 < jd[k] ? ld_stream_i32(p.colidx + rs + 1, pol) : -1;
                    nv2[k] = rs + 1 < jd[k] ? ld_stream_f64(p.val + rs + 1, pol) : 0.0;
                    ls[k] = 0.0;
                    st_load |= 1u << k;
                    prog = true;
                }
                nxt += min(__popc(fm), avail);
                if (nxt >= rows_cur) {
                    // sub-chunk fully assigned: switch to the prefetched one, prefetch the next
                    cp_async_wait_all();
                    __syncwarp();
                    s_cur = s_nxt;
                    cb ^= 1;
                    nxt = 0;
                    s_nxt = s_cur < p.n ? next_sub() : p.n;
                    load_sub(s_nxt, cb ^ 1);
                } else {
                    break;
                }
            }
        }
        // ---- one global poll per ACTIVE slot
        unsigned long long w0[K], w1[K];
#pragma unroll
        for (int k = 0; k < K; ++k) {
            w0[k] = 0;
            w1[k] = 0;
            if ((st_act >> k & 1u) && nc[k] >= 0) poll1<PROTO>(pp, nc[k], w0[k], w1[k]);
        }
        // ---- ACTIVE: consume the ready dependency or publish at the diagonal
#pragma unroll
        for (int k = 0; k < K; ++k) {
            if (!(st_act >> k & 1u)) continue;
            bool fin = nc[k] < 0;
            if (!fin && ready1<PROTO>(w0[k], w1[k], epoch)) {
                if (p.trace) p.trace[p.n + ri[k]] = globaltimer_ns();
                ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], value1<PROTO>(pp, nc[k], w0[k], w1[k])));
                ++j[k];
                nc[k] = nc2[k];
                nv[k] = nv2[k];
                nc2[k] = j[k] + 1 < jd[k] ? ld_stream_i32(p.colidx + j[k] + 1, pol) : -1;
                nv2[k] = j[k] + 1 < jd[k] ? ld_stream_f64(p.val + j[k] + 1, pol) : 0.0;
                fin = nc[k] < 0;
                prog = true;
            }
            if (fin) {
                Diag dg;
                dg.d = dd[k];
                dg.r = rr[k];
                publish<PROTO>(pp, nocta, ri[k], dg.div(__dsub_rn(bi[k], ls[k])), epoch);
                ri[k] = -1;
                st_act &= ~(1u << k);
                prog = true;
            }
        }
        // ---- done when no chunk is left and every slot is free
        bool busy = s_cur < p.n;
#pragma unroll
        for (int k = 0; k < K; ++k) busy |= ri[k] >= 0;
        if (!__ballot_sync(FULL, busy)) break;
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
    cp_async_wait_all();
}

}  // namespace sptrsv_dev
