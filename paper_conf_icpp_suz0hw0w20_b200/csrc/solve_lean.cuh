// solve_lean.cuh -- ENGINE_LEAN: the minimal-latency one-shot kernel for
// all-thread-level plans (short rows, the paper's target regime PAPER.md:188-192).
//
// Alg.5 with everything that is not the method trimmed off
// the per-CTA critical path, because for rows of 2-4 entries the method's own
// work is a few instructions and the solve is bound by how fast rows ENTER the
// machine (measured: a 1M-row diagonal solve, no dependencies at all, took 26 us
// in the staged engine vs a 14 us streaming floor):
//   * the CTA ticket (forward progress, solve.cuh cta_ticket) is overlapped
//     with a SPECULATIVE load of the rows the CTA gets when its ticket equals
//     blockIdx.x (the common case; otherwise the rows are re-loaded);
//   * no shared-memory staging and no in-CTA x copy: each lane loads its row's
//     bounds, b_i, L_ii and first two entries straight into registers;
//   * small register footprint (higher occupancy = more rows in flight).
// The poll / consume / publish protocol (FLAGS or FUSED), the verified division
// and the lean wait are the shared ones from solve.cuh.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

constexpr int kLeanCta = 256;

// A lane's row once its second-level loads are issued: the off-diagonals [lo, hi) walked from j
// (earliest-solved first), the next two dependencies (column, value) and L_ii.
struct LeanRow {
    int lo, hi, j, nc, nc2;
    double nv, nv2, dv;
};

// Second-level loads of row i with bounds [rs, re): L_ii and the first two dependencies.  Split from
// lean_rows so that k_solve_lean can issue them BEFORE the CTA barrier that waits for the start
// ticket: the ticket's same-address atomic then overlaps both load phases.
template <bool UPPER, bool UNIT>
__device__ __forceinline__ LeanRow lean_load(const SolveParams &p, bool act, int rs, int re, uint64_t pol) {
    // off-diagonal entries [lo, hi); the diagonal is last (lower), first (upper) or implicit
    // (unit).  They are consumed earliest-solved first: ascending for lower (Alg.1 l.3-4),
    // DESCENDING for upper (G25) -- the nearest, latest dependency is waited for last.
    LeanRow r;
    r.lo = (UPPER && !UNIT) ? rs + 1 : rs;
    r.hi = (UPPER || UNIT) ? re : re - 1;
    constexpr int dir = UPPER ? -1 : 1;
    auto inr = [&](int k) { return UPPER ? k >= r.lo : k < r.hi; };
    r.j = UPPER ? r.hi - 1 : r.lo;
    r.dv = (act && !UNIT) ? ld_stream_f64(p.val + (UPPER ? rs : re - 1), pol) : 1.0;
    r.nc = (act && inr(r.j)) ? ld_stream_i32(p.colidx + r.j, pol) : -1;
    r.nv = (act && inr(r.j)) ? ld_stream_f64(p.val + r.j, pol) : 0.0;
    r.nc2 = (act && inr(r.j + dir)) ? ld_stream_i32(p.colidx + r.j + dir, pol) : -1;
    // the second dependency's VALUE is preloaded too: consuming both dependencies in one pass
    // (the common case when the earlier one is long solved) then never waits on a reload
    r.nv2 = (act && inr(r.j + dir)) ? ld_stream_f64(p.val + r.j + dir, pol) : 0.0;
    return r;
}

// One warp, one row per lane (Alg.5 l.3-18): lane's row i (act: i is a real row), b_i and its
// second-level loads (lean_load) already issued.  Returns when every lane of the warp has
// published, or on abort.  Shared by k_solve_lean and the f4 list kernel (solve_tri.cuh).
template <int PROTO, bool UPPER, bool UNIT>
__device__ __forceinline__ void lean_rows(SolveParams &p, int i, bool act, const LeanRow &lr, double bi,
                                          uint32_t epoch, int lane, uint64_t pol, double *xout = nullptr) {
    const int lo = lr.lo, hi = lr.hi;
    constexpr int dir = UPPER ? -1 : 1;
    auto inr = [&](int k) { return UPPER ? k >= lo : k < hi; };
    int j = lr.j, nc = lr.nc, nc2 = lr.nc2;
    double nv = lr.nv, nv2 = lr.nv2;
    const double dv = lr.dv;
    Diag dg;
    dg.init(dv);
    if (p.trace && act && nc != -2) p.trace[2 * (size_t)p.n + i] = globaltimer_ns();  // loads landed
    double ls = 0.0;
    bool done = !act;
    Cta nocta;
    nocta.R0 = nocta.R1 = 0;
    nocta.xc = nullptr;
    nocta.xc_s = 0;
    p.local = 0;  // no in-CTA x copy in this engine
    uint32_t backoff = p.backoff_min, idle = 0;
    // advance past a consumed dependency: the 2nd becomes the next, prefetch the 3rd
    auto advance = [&]() {
        j += dir;
        nc = nc2;
        nv = nv2;
        const bool more = inr(j + dir);
        nc2 = more ? ld_stream_i32(p.colidx + j + dir, pol) : -1;
        nv2 = more ? ld_stream_f64(p.val + j + dir, pol) : 0.0;
    };
    while (true) {
        bool prog = false;
        if (!done) {
            if (nc < 0) {  // reached the diagonal (Alg.5 l.12-16)
                const double xi = UNIT ? __dsub_rn(bi, ls) : dg.div(__dsub_rn(bi, ls));
                publish<PROTO>(p, nocta, i, xi, epoch);
                if (xout) *xout = xi;
                done = true;
                prog = true;
            } else {
                // poll the next two dependencies together, consume the ready prefix in row order
                unsigned long long a0, a1, c0 = 0, c1 = 0;
                poll1<PROTO>(p, nc, a0, a1);
                const int cc2 = p.poll_one ? -1 : nc2;
                if (cc2 >= 0) poll1<PROTO>(p, cc2, c0, c1);
                if (ready1<PROTO>(a0, a1, epoch)) {
                    if (p.trace) p.trace[p.n + i] = globaltimer_ns();
                    ls = __dadd_rn(ls, __dmul_rn(nv, value1<PROTO>(p, nc, a0, a1)));
                    advance();
                    prog = true;
                    if (cc2 >= 0 && ready1<PROTO>(c0, c1, epoch)) {
                        ls = __dadd_rn(ls, __dmul_rn(nv, value1<PROTO>(p, cc2, c0, c1)));
                        advance();
                    }
                    if (nc < 0) {
                        const double xi = UNIT ? __dsub_rn(bi, ls) : dg.div(__dsub_rn(bi, ls));
                publish<PROTO>(p, nocta, i, xi, epoch);
                if (xout) *xout = xi;
                        done = true;
                    }
                }
            }
        }
        if (!__ballot_sync(FULL, !done)) break;
        if (__ballot_sync(FULL, prog)) {
            backoff = p.backoff_min;
            idle = 0;
            if (p.poll_gap) nanosleep_ns(p.poll_gap);
            continue;
        }
        if (backoff) nanosleep_ns(backoff);
        backoff = min(max(backoff * 2u, 32u), p.backoff_max);
        if ((++idle & 63u) == 0) {
            uint32_t ab = 0;
            if (lane == 0) {
                if (p.spin_limit && idle >= p.spin_limit) {
                    atomicCAS(&p.st->error.v, 0u, kErrTimeout);
                    st_relaxed_u32(&p.st->abort.v, 1u);
                }
                ab = ld_relaxed_u32(&p.st->abort.v);
            }
            if (__shfl_sync(FULL, ab, 0)) break;
        }
    }
}

// UPPER / UNIT: upper-triangular rows (diagonal first, dependencies
// j > i) are taken in REVERSE order -- logical row r is row n-1-r, so the ticket
// order is again a topological order; UNIT: the diagonal is implicitly 1 and
// not stored.
template <int PROTO, int MINB, bool UPPER = false, bool UNIT = false, int CT = kLeanCta>
__global__ void __launch_bounds__(CT, MINB) k_solve_lean(SolveParams p) {
    __shared__ uint32_t s_blk, s_epoch;
    const int tid = threadIdx.x;
    const int lane = tid & 31;
    const uint64_t pol = policy_evict_first();
    // ---- speculative first-level loads for logical block == blockIdx.x (the common case), overlapped
    // with the start ticket (round 2 also issued the second-level loads before the barrier: c5 53 ->
    // 60 us, reverted)
    int i = (int)blockIdx.x * CT + tid;
    if (UPPER) i = p.n - 1 - i;
    int rs = 0, re = 1;
    double bi = 0.0;
    const bool bgate = p.bflag != nullptr;  // b still arriving in chunks (sptrsv_solve_host)
    if (i >= 0 && i < p.n) {
        if (p.trace) p.trace[3 * (size_t)p.n + 3 + i] = globaltimer_ns();  // CTA entry
        rs = ld_stream_i32(p.rowptr + i, pol);
        re = ld_stream_i32(p.rowptr + i + 1, pol);
        if (!bgate) bi = ld_b(p, i, pol);
    }
    if (tid == 0) {
        if (p.trace) {
            atomicMin(&p.trace[3 * (size_t)p.n], globaltimer_ns());                  // first CTA entry
            atomicAdd(&p.trace[3 * (size_t)p.n + 2], 1ull);                          // CTAs started
        }
        cta_ticket(p, s_blk, s_epoch);
        if (bgate) {  // wait until the b chunks of this CTA's (physical) rows have landed
            const int lr0 = (int)s_blk * CT, lr1 = min(p.n, lr0 + CT);
            wait_b_chunks(p, UPPER ? p.n - lr1 : lr0, UPPER ? p.n - lr0 : lr1);
        }
    }
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    if (s_blk != blockIdx.x) {  // rare: re-load for the block the ticket assigned
        i = (int)s_blk * CT + tid;
        if (UPPER) i = p.n - 1 - i;
        rs = 0, re = 1, bi = 0.0;
        if (i >= 0 && i < p.n) {
            rs = ld_stream_i32(p.rowptr + i, pol);
            re = ld_stream_i32(p.rowptr + i + 1, pol);
            bi = ld_b(p, i, pol);
        }
    } else if (bgate && i >= 0 && i < p.n) {
        bi = ld_b(p, i, pol);
    }
    const bool act = i >= 0 && i < p.n;
    lean_rows<PROTO, UPPER, UNIT>(p, i, act, lean_load<UPPER, UNIT>(p, act, rs, re, pol), bi, epoch, lane, pol);
    if (p.trace && lane == 0) atomicMax(&p.trace[3 * (size_t)p.n + 1], globaltimer_ns());  // last warp exit
    if (p.x_host) {
        // sptrsv_solve_host: the CTA's finished rows go to pinned host memory over PCIe as one
        // contiguous, coalesced block per CTA (8-byte per-row publishes would each be a TLP),
        // overlapping the device->host transfer with the rest of the solve
        __syncthreads();
        const int lr0 = (int)s_blk * CT, lr1 = min(p.n, lr0 + CT);
        if (lr0 < lr1) {
            const int a = UPPER ? p.n - lr1 : lr0, e = UPPER ? p.n - lr0 : lr1;
            for (int r = a + tid; r < e; r += CT) p.x_host[r] = __ldcg(p.x + r);
        }
    }
}


// ENGINE_LEANP: LEAN with PERSISTENT warps and a software pipeline.  The grid is
// exactly what fits on the device at once (cooperative launch: every CTA is co-resident), CTA c
// (its logical id from the start ticket) owns blocks c, c + G, c + 2G, ... of 256 logical rows, and
// warp w of the CTA owns the 32-row slice w of each: a static round-robin that needs no work
// tickets.  Each warp keeps three chunks in flight: the first-level loads (rowptr, b) of chunk k+2,
// the second-level loads (L_ii, first two dependencies) of chunk k+1 and the solve of chunk k, so the
// two dependent DRAM round trips of a chunk overlap the previous chunk's dependency waits instead of
// adding to them.  Forward progress: the lowest unsolved row's chunk is the current chunk of its
// warp (the warp's earlier chunks are lower, hence solved) and every warp is resident.
template <int PROTO, int MINB, bool UPPER = false, bool UNIT = false>
__global__ void __launch_bounds__(kLeanCta, MINB) k_solve_leanp(SolveParams p) {
    constexpr int CT = kLeanCta;
    __shared__ uint32_t s_blk, s_epoch;
    const int tid = threadIdx.x;
    const int lane = tid & 31, warp = tid >> 5;
    const uint64_t pol = policy_evict_first();
    if (tid == 0) cta_ticket(p, s_blk, s_epoch);
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const long long G = p.grid, c = s_blk;
    const long long nblk = ((long long)p.n + CT - 1) / CT;
    // logical row of this lane in its k-th chunk (>= n: past the end)
    auto row_of = [&](long long k) -> long long { return (c + k * G) * CT + warp * 32 + lane; };
    auto phys = [&](long long r) -> int { return UPPER ? p.n - 1 - (int)r : (int)r; };
    auto first = [&](long long k, int &rs, int &re, double &bi) {
        const long long r = row_of(k);
        rs = 0, re = 1, bi = 0.0;
        if (r < p.n) {
            const int i = phys(r);
            rs = ld_stream_i32(p.rowptr + i, pol);
            re = ld_stream_i32(p.rowptr + i + 1, pol);
        }
        // (with sptrsv_solve_host's chunked b, b is loaded just before the chunk's solve instead: a
        // prefetch would wait for b two chunks ahead of the solve)
        if (r < p.n && !p.bflag) bi = ld_b(p, phys(r), pol);
    };
    auto gated_b = [&](long long k, double &bi) {  // lane 0 waits for the chunk(s) of the warp's rows
        const long long r = row_of(k), r0 = r - lane;
        if (lane == 0 && r0 < p.n) {
            const int a = (int)r0, e = (int)min((long long)p.n, r0 + 32);
            wait_b_chunks(p, UPPER ? p.n - e : a, UPPER ? p.n - a : e);
        }
        __syncwarp();
        if (r < p.n) bi = ld_b(p, phys(r), pol);
    };
    if (c >= nblk) return;
    int rs1, re1, rs2, re2;
    double bi0, bi1, bi2;
    first(0, rs1, re1, bi0);
    bool act0 = row_of(0) < p.n;
    LeanRow lr0 = lean_load<UPPER, UNIT>(p, act0, rs1, re1, pol);
    first(1, rs1, re1, bi1);
    for (long long k = 0; c + k * G < nblk; ++k) {
        const bool act1 = row_of(k + 1) < p.n;
        const LeanRow lr1 = lean_load<UPPER, UNIT>(p, act1, rs1, re1, pol);  // chunk k+1: second level
        first(k + 2, rs2, re2, bi2);                                           // chunk k+2: first level
        const long long r0 = row_of(k);
        if (p.bflag) gated_b(k, bi0);
        double xi = 0.0;
        lean_rows<PROTO, UPPER, UNIT>(p, r0 < p.n ? phys(r0) : 0, act0, lr0, bi0, epoch, lane, pol, &xi);
        // sptrsv_solve_host: the warp's finished rows to pinned host memory (UVA), 256 contiguous bytes,
        // from the registers (no read-back of x on the pipeline)
        if (p.x_host && act0) p.x_host[phys(r0)] = xi;
        lr0 = lr1;
        act0 = act1;
        bi0 = bi1;
        rs1 = rs2, re1 = re2, bi1 = bi2;
    }
}

}  // namespace sptrsv_dev
