// solve_chain.cuh -- ENGINE_CHAIN: warp-sequential resolution of in-warp dependency chains.
//
// The same per-row method as every engine -- Alg.5 Writing-First for
// thread-level rows: stream the row, consume ready
// dependencies in row order, divide at the diagonal, publish -- but with the
// dependencies that fall INSIDE a warp's own rows resolved in registers instead
// of through a flag / record round trip.  That is the shape of the paper's
// "pure chain" and grid-wavefront regimes (bidiagonal and 5-point lower
// factors: row i depends on i-1), where the one-shot engine paid ~0.3 us per
// in-warp hop (shared-memory local rounds) and the record protocol ~0.5 us.
//
// A warp owns R = 32K consecutive rows r0 .. r0+R-1 (lane l owns r0 + l + 32k).
// A row's off-diagonals split, by the sorted CSR order, into EXTERNAL ones
// (col < r0, other warps: global FUSED / FLAGS protocol) followed by INTERNAL
// ones (col in [r0, i), rows of this warp).  Each pass:
//   A. external: every unfinished row whose next entry is external issues a poll
//      (K polls per lane in flight while B and C run; consumed in D);
//   B. catch-up: rows whose next entries are internal and already finalized
//      read them from the warp's shared-memory copy s_x;
//   C. chain: from the first unfinalized row s, while row s has no external
//      entry left, its owner divides and publishes, the value is broadcast
//      with one __shfl_sync, and every row whose next entry is column r0+s
//      consumes it -- one step per row, no memory round trip on the chain;
//   D. the polls of A are consumed (ready ones advance their row).
// Accumulation stays in row order with separately rounded mul and add (external
// entries precede internal ones in a sorted row), so x is bit-identical to
// Alg.1, like every thread-level path.  Forward progress: a
// row only waits on external rows (earlier warps / CTAs, which started first by
// the CTA ticket) or on earlier rows of its own warp, finalized in order.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

constexpr int kChainCta = 128;  // 4 warps
constexpr int kChainEPR = 4;    // staged CSR entries per row (a longer slice reads global memory)

__host__ __device__ constexpr int chain_warp_smem_bytes(int K) {
    // s_val [32K*EPR] f64 | s_x [32K] f64 | f_b, f_d, f_r, f_ls, f_v [32K] f64 |
    // s_col [32K*EPR] i32 | f_has [32K] i32 | s_rp [32K+1] i32   (16-B multiple)
    return ((8 * 32 * K * kChainEPR + 8 * 32 * K + 5 * 8 * 32 * K + 4 * 32 * K * kChainEPR + 4 * 32 * K +
             4 * (32 * K + 1)) + 15) / 16 * 16;
}

// UPPER / UNIT (G25): the warp owns LOGICAL rows r0 .. r0+R-1, logical row
// r = physical row n-1-r for upper handles, so the ticket order stays a topological order.  All
// the chain logic runs on logical indices (dependencies: logical column < logical row); a row's
// off-diagonals are walked earliest-solved first (descending physical column for upper), its
// diagonal is the first entry (upper), the last (lower) or implicit 1 (unit).  Loads of CSR
// entries, polls and publication use physical indices.
// SAFE (SPTRSV_OPT_CHAIN_DIV = 1): the fast loop proves every quotient before using it (Diag::exact
// in the loop condition, +~25 cycles per chain step).  Otherwise (default) the fast loop runs the
// Markstein candidate at full speed and the rows of each run are proven right after the run, all
// lanes in parallel; a candidate that is not RN(a/d) -- never observed --
// aborts the solve with kErrInexact, sptrsv_check reports SPTRSV_ERR_INEXACT and switches the
// handle to SAFE, so no solve ever returns an unproven quotient.
template <int PROTO, int K, bool UPPER = false, bool UNIT = false, bool SAFE = false>
__global__ void __launch_bounds__(256, K == 1 ? 4 : 3) k_solve_chain(SolveParams p) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint32_t s_blk, s_epoch;
    constexpr int RT = 32 * K;
    constexpr int ECAP = RT * kChainEPR;
    const int warps = blockDim.x >> 5;
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        cta_ticket(p, s_blk, s_epoch);
        if (p.bflag) {  // sptrsv_solve_host: this CTA's b chunks (physical rows)
            const int lr0 = (int)s_blk * (int)(blockDim.x >> 5) * 32 * K;
            const int lr1 = min(p.n, lr0 + (int)(blockDim.x >> 5) * 32 * K);
            wait_b_chunks(p, UPPER ? p.n - lr1 : lr0, UPPER ? p.n - lr0 : lr1);
        }
    }
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const int r0 = ((int)s_blk * warps + warp) * RT;
    if (r0 >= p.n) return;
    const int rows = min(RT, p.n - r0);
    const uint64_t pol = policy_evict_first();
    p.local = 0;  // no CTA-wide x copy in this engine (publish() skips it)
    Cta nocta;
    nocta.R0 = nocta.R1 = 0;
    nocta.xc = nullptr;
    nocta.xc_s = 0;
    unsigned char *wsm = smem + (size_t)warp * chain_warp_smem_bytes(K);
    double *s_val = reinterpret_cast<double *>(wsm);
    double *s_x = s_val + ECAP;
    double *f_b = s_x + RT, *f_d = f_b + RT, *f_r = f_d + RT, *f_ls = f_r + RT, *f_v = f_ls + RT;
    int32_t *s_col = reinterpret_cast<int32_t *>(f_v + RT);
    int32_t *f_has = s_col + ECAP;
    int32_t *s_rp = f_has + RT;
    // logical <-> physical (upper: reversed); s_rp holds the slice's rowptr in PHYSICAL order
    const int p0 = UPPER ? p.n - r0 - rows : r0;                  // first physical row of the slice
    auto phys = [&](int lr) { return UPPER ? p.n - 1 - lr : lr; };  // logical row / column -> physical
    auto slot = [&](int t) { return UPPER ? rows - 1 - t : t; };    // warp row t -> s_rp index
    constexpr int dir = UPPER ? -1 : 1;                             // entry walk, earliest-solved first
    // ---- stage rowptr, b, then the warp's contiguous CSR slice (coalesced)
    double bk[K];  // staging only: the rows' constants live in smem (f_b, f_d, f_r) afterwards
#pragma unroll
    for (int k = 0; k <= K; ++k) {
        const int idx = lane + 32 * k;
        if (idx <= rows) s_rp[idx] = ld_stream_i32(p.rowptr + p0 + idx, pol);
    }
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const int idx = lane + 32 * k;
        bk[k] = idx < rows ? ld_b(p, phys(r0 + idx), pol) : 0.0;
    }
    __syncwarp();
    const int base = s_rp[0];
    const int len = s_rp[rows] - base;
    const bool staged = len <= ECAP;  // warp-uniform
    if (staged) {
#pragma unroll 4
        for (int e = lane; e < len; e += 32) {
            s_col[e] = ld_stream_i32(p.colidx + base + e, pol);
            s_val[e] = ld_stream_f64(p.val + base + e, pol);
        }
    }
    __syncwarp();
    auto col_at = [&](int jj) -> int { return staged ? s_col[jj - base] : ld_stream_i32(p.colidx + jj, pol); };
    auto val_at = [&](int jj) -> double { return staged ? s_val[jj - base] : ld_stream_f64(p.val + jj, pol); };
    // ---- per-row state: cursor j, end je (one step past the last off-diagonal: the diagonal,
    // or the row's edge for unit forms), next LOGICAL column / value, partial sum
    int j[K], je[K], nc[K];
    double nv[K], ls[K], xm[K];
    unsigned done = 0;  // bit k: row k of this lane finalized (or not a row)
    auto lcol = [&](int jj) { return UPPER ? p.n - 1 - col_at(jj) : col_at(jj); };
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const int idx = lane + 32 * k;
        const bool a = idx < rows;
        const int rs = a ? s_rp[slot(idx)] : 0, re = a ? s_rp[slot(idx) + 1] : 0;
        // lower: [rs, re-1) ascending, diagonal re-1; upper: (rs, re) descending, diagonal rs;
        // unit: every stored entry is an off-diagonal
        j[k] = UPPER ? re - 1 : rs;
        je[k] = UPPER ? (UNIT ? rs - 1 : rs) : (UNIT ? re : re - 1);
        if (!a) j[k] = je[k] = 0;
        nc[k] = (a && j[k] != je[k]) ? lcol(j[k]) : -1;
        nv[k] = (a && j[k] != je[k]) ? val_at(j[k]) : 0.0;
        ls[k] = 0.0;
        xm[k] = 0.0;
        Diag dg;
        dg.init((a && !UNIT) ? val_at(UPPER ? rs : re - 1) : 1.0);
        if (!a) done |= 1u << k;
        f_b[idx] = bk[k];  // the rows' constants (both chain paths read them from smem)
        f_d[idx] = dg.d;
        f_r[idx] = dg.r;
    }
    auto advance = [&](int k) {
        j[k] += dir;
        const bool more = j[k] != je[k];
        nc[k] = more ? lcol(j[k]) : -1;
        nv[k] = more ? val_at(j[k]) : 0.0;
    };
    const bool tracing = p.trace != nullptr;
    int s = 0;  // next row (warp-relative) to finalize; rows < s are published
    uint32_t backoff = p.backoff_min, idle = 0;
    // the fast loop's rows of the current pass, proven after the run (!SAFE)
    int vf0 = 0, vf1 = 0;
    while (true) {
        bool prog = false;
        // ---- A. external dependencies: one poll per unfinished row, K in flight
        unsigned long long w0[K], w1[K];
        unsigned gm = 0;
#pragma unroll
        for (int k = 0; k < K; ++k) {
            w0[k] = 0;
            w1[k] = 0;
            if (!(done >> k & 1u) && nc[k] >= 0 && nc[k] < r0) {
                gm |= 1u << k;
                poll1<PROTO>(p, phys(nc[k]), w0[k], w1[k]);
            }
        }
        // ---- consume the ready polls
#pragma unroll
        for (int k = 0; k < K; ++k) {
            if ((gm >> k & 1u) && ready1<PROTO>(w0[k], w1[k], epoch)) {
                if (p.trace) p.trace[p.n + phys(r0 + lane + 32 * k)] = globaltimer_ns();
                ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], value1<PROTO>(p, phys(nc[k]), w0[k], w1[k])));
                advance(k);
                prog = true;
            }
        }
        // ---- B. internal entries finalized in an earlier run: read the warp's smem copy
        __syncwarp();
#pragma unroll
        for (int k = 0; k < K; ++k) {
            while (!(done >> k & 1u) && nc[k] >= r0 && nc[k] < r0 + s) {
                ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], s_x[nc[k] - r0]));
                advance(k);
                prog = true;
            }
        }
        // ---- C. the chain: rows with no external entry left, finalized in row order
        unsigned long long ok = 0;  // bit t: warp row t is done or has only internal entries / the diagonal left
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const bool rdy = (done >> k & 1u) || nc[k] < 0 || nc[k] >= r0;
            ok |= (unsigned long long)__ballot_sync(FULL, rdy) << (32 * k);
        }
        const int s0 = s;
        const unsigned long long nok = ~ok >> s;
        const int run_end = min(rows, nok ? s + __ffsll((long long)nok) - 1 : 64);
        // One step per row: the owner divides (Diag: the Markstein step, RN(a/d) inside the
        // guard) and its value is broadcast by one __shfl_sync to the rows that consume it.
        // FUSED publishes each value at once (one 16-byte record store, the only per-step
        // store); x, the smem copy and FLAGS publication are written per run, coalesced.
        // Fast path (bidiagonal chains, grid west neighbours): when every row of the run has
        // at most ONE internal entry left and it is the previous row, the run is the scalar
        // recurrence x_t = (b_t - (ls_t + v_t x_{t-1})) / d_t.  All 32 lanes then evaluate it
        // REDUNDANTLY from the run's operands in shared memory (broadcast loads): no shuffle and
        // no lane-to-lane hop on the chain, only its dependent fp64 operations.  Same
        // operations in the same order as Alg.1 (mul, add, sub, division), so bit-exact.
        bool el = true;
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const int t = lane + 32 * k;
            if (!(done >> k & 1u) && t >= s && t < run_end) {
                const bool none = nc[k] < 0;
                const bool prev = nc[k] == r0 + t - 1 && j[k] + dir == je[k];
                el = el && (none || (prev && t > s));
                f_ls[t] = ls[k];
                f_v[t] = prev ? nv[k] : 0.0;
                f_has[t] = prev ? 1 : 0;
            }
        }
        vf0 = vf1 = s;
        if (run_end > s && __all_sync(FULL, el)) {
            __syncwarp();
            double xp = 0.0;  // x of row t - 1 (read only when row t has that entry)
            // operands of row t are loaded one iteration ahead, off the dependency chain
            double lsv = f_ls[s], bv = f_b[s], vv = f_v[s], dv = f_d[s], rv = f_r[s];
            int hv = f_has[s];
            int t = s;
            for (; t < run_end; ++t) {
                const int tn = min(t + 1, run_end - 1);
                const double lsn = f_ls[tn], bn = f_b[tn], vn = f_v[tn], dn = f_d[tn], rn = f_r[tn];
                const int hn = f_has[tn];
                const double u = hv ? __dadd_rn(lsv, __dmul_rn(vv, xp)) : lsv;
                const double a = __dsub_rn(bv, u);
                Diag g;
                g.d = dv;
                g.r = rv;
                const double q = g.cand(a);
                // guard (Diag::ok) in integer ops, warp-uniform here (every lane holds the same a).  A
                // failure LEAVES the fast loop instead of branching around an in-loop __ddiv_rn: the
                // loop body then has no reconvergence point, and the guard resolves from a while the
                // Markstein step is still in flight (chain step ~140 -> ~90 cycles, chainstep.cu)
                if (__builtin_expect(!(Diag::in_range(a) && __double2hiint(rv) != 0 &&
                                       (!SAFE || Diag::exact(a, dv, q))), 0))
                    break;
                if (!SAFE) f_ls[t] = a;  // the numerator, for the proof after the run (own store, all lanes)
                const int owner = t & 31, kk = t >> 5;
                const bool mine = lane == owner;
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    const bool mk = mine && kk == k;
                    xm[k] = mk ? q : xm[k];
                    done |= mk ? (1u << k) : 0u;
                    nc[k] = mk ? -1 : nc[k];
                }
                if (PROTO == PROTO_FUSED) {  // the owner's record: one predicated store, no branch
                    unsigned long long bits = (unsigned long long)__double_as_longlong(q);
                    bits = bits == kSentinel ? kCanonNaN : bits;
                    const unsigned long long e = (unsigned long long)epoch << 32;
                    st_relaxed_v2_u64_if(mine, p.rec + 2 * (size_t)phys(r0 + t), e | (bits & 0xffffffffull), e | (bits >> 32));
                    if (tracing) st_u64_if(mine, p.trace + phys(r0 + t), globaltimer_ns());
                }
                xp = q;
                lsv = lsn, bv = bn, vv = vn, dv = dn, rv = rn, hv = hn;
            }
            vf1 = t;
            if (t < run_end && hv) {
                // the guard failed at row t: the exact loop below finishes the run from t.  Row t's
                // previous-row entry is consumed first, by its owner, with the same mul and add as the
                // fast step (so the sum stays bit-identical to Alg.1)
                const int owner = t & 31, kk = t >> 5;
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    if (lane == owner && kk == k) {
                        ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], xp));
                        advance(k);
                    }
                }
            }
            s = t;
        }
#pragma unroll
        for (int k = 0; k < K; ++k) {  // rows r0 + 32k .. r0 + 32k + 31: owner lane = s - 32k
            const int hi = min(run_end, 32 * (k + 1));
            for (; s < hi; ++s) {
                const int owner = s - 32 * k;
                Diag g;
                g.d = f_d[s];
                g.r = f_r[s];
                const double a = __dsub_rn(f_b[s], ls[k]);
                double q = g.cand(a);
                const int bad = !g.ok(a, q);
                double xv = __shfl_sync(FULL, q, owner);
                if (__shfl_sync(FULL, bad, owner)) {  // warp-uniform, rare: outside the guard
                    q = __ddiv_rn(a, g.d);
                    xv = __shfl_sync(FULL, q, owner);
                }
                const bool mine = lane == owner;
                xm[k] = mine ? q : xm[k];
                done |= mine ? (1u << k) : 0u;
                if (PROTO == PROTO_FUSED) {
                    unsigned long long bits = (unsigned long long)__double_as_longlong(q);
                    bits = bits == kSentinel ? kCanonNaN : bits;  // same canonicalisation as publish()
                    const unsigned long long e = (unsigned long long)epoch << 32;
                    st_relaxed_v2_u64_if(mine, p.rec + 2 * (size_t)phys(r0 + s), e | (bits & 0xffffffffull), e | (bits >> 32));
                    if (tracing) st_u64_if(mine, p.trace + phys(r0 + s), globaltimer_ns());
                }
                const int cs = r0 + s;
#pragma unroll
                for (int m = 0; m < K; ++m) {  // done rows hold nc = -1
                    const bool c = nc[m] == cs;
                    const double t = __dadd_rn(ls[m], __dmul_rn(nv[m], xv));
                    ls[m] = c ? t : ls[m];
                    if (c) advance(m);
                }
            }
        }
        if (!SAFE && !UNIT && vf1 > vf0) {
            // the proof of the fast loop's quotients (Diag::exact), one row per owner lane: row t's
            // numerator is f_ls[t], its quotient the owner's xm
            bool bad = false;
#pragma unroll
            for (int k = 0; k < K; ++k) {
                const int t = lane + 32 * k;
                if (t >= vf0 && t < vf1) bad |= (p.chain_div == 2) | !Diag::exact(f_ls[t], f_d[t], xm[k]);
            }
            if (__any_sync(FULL, bad)) {
                if (lane == 0) {
                    atomicCAS(&p.st->error.v, 0u, kErrInexact);
                    st_relaxed_u32(&p.st->abort.v, 1u);
                }
                return;
            }
        }
        if (s > s0) {
            // the run's x (output), the smem copy for later in-warp consumers and, for FLAGS, the
            // release pattern (PTX model, G6): x stores, one gpu-scope fence, relaxed flags
#pragma unroll
            for (int k = 0; k < K; ++k) {
                const int t = lane + 32 * k;
                if (t >= s0 && t < s) {
                    p.x[phys(r0 + t)] = xm[k];
                    s_x[t] = xm[k];
                    if (PROTO == PROTO_FLAGS && p.trace) p.trace[phys(r0 + t)] = globaltimer_ns();
                }
            }
            if (PROTO == PROTO_FLAGS) {
                fence_acq_rel_gpu();
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    const int t = lane + 32 * k;
                    if (t >= s0 && t < s) st_relaxed_u32(p.flags + phys(r0 + t), epoch);
                }
            }
        }
        if (s >= rows) {
            if (p.x_host) {  // sptrsv_solve_host: the warp's rows to pinned host memory, coalesced
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    const int t = lane + 32 * k;
                    if (t < rows) p.x_host[phys(r0 + t)] = xm[k];
                }
            }
            break;
        }
        if (s > s0) prog = true;
        if (__ballot_sync(FULL, prog)) {
            backoff = p.backoff_min;
            idle = 0;
            continue;
        }
        // ---- lean wait: nothing moved, so every unfinished row is blocked on an external entry;
        // re-poll only those (a few instructions per round instead of a full pass) until one is
        // ready, then consume it and run a full pass
        bool woke = false;
        while (!woke) {
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
                if (__shfl_sync(FULL, ab, 0)) return;
            }
            bool got = false;
#pragma unroll
            for (int k = 0; k < K; ++k) {
                if (!(done >> k & 1u) && nc[k] >= 0 && nc[k] < r0) {
                    unsigned long long a0, a1;
                    poll1<PROTO>(p, phys(nc[k]), a0, a1);
                    if (ready1<PROTO>(a0, a1, epoch)) {
                        if (p.trace) p.trace[p.n + phys(r0 + lane + 32 * k)] = globaltimer_ns();
                        ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], value1<PROTO>(p, phys(nc[k]), a0, a1)));
                        advance(k);
                        got = true;
                    }
                }
            }
            woke = __ballot_sync(FULL, got) != 0;
        }
        backoff = p.backoff_min;
    }
}

}  // namespace sptrsv_dev
