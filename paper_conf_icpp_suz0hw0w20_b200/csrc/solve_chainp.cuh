// solve_chainp.cuh -- ENGINE_CHAINP: in-warp dependency chains, each chain warp paired with a POLLER warp.
//
// The per-row method is Alg.5's: consume a row's dependencies in row order,
// divide at the diagonal, publish x_i.  Like the round-1 CHAIN engine, the dependencies that fall
// inside a pair's own R = 32K consecutive rows are resolved on chip instead of through a ready
// record, which is what grid wavefronts and pure chains need (row i depends on i-1).  What changes
// is who waits for the EXTERNAL ones (columns before the pair's first row) and how many rows one
// SM holds:
//   POLLER  owns the rows' external entries.  It polls a window of the 64 lowest rows that still
//           have one (two rows per lane; Alg.5 l.8), consumes the ready ones in row order (l.9)
//           and, when a row has no external entry left, writes the row's partial sum to shared
//           memory and sets the row's bit in a ready mask.
//   CHAIN   finalizes rows in order: it waits (in shared memory only) for the next row's bit,
//           adds the row's internal entries -- earlier rows of this pair, already final --
//           divides (Alg.5 l.13) and publishes (l.14-16).  All 32 lanes evaluate the chain
//           redundantly from shared-memory operands, so a step is its dependent fp64 operations:
//           no shuffle, no vote, no global memory round trip.
// The chain warp never waits on L2 except to publish, and the poller never waits on the chain.
//
// Why it matters (c3, the 2048^2 grid factor): rows enter in ticket (row)
// order, so every grid line below the wavefront that has started holds its CTAs resident while it
// waits; a line can only start when enough earlier rows have retired.  The steady-state lag per
// line is then about (line span) x 1024 / (resident rows), so the engine is built for many
// resident rows per SM (all per-row state in shared memory, ~76 B per row, 32K rows per pair)
// and a short line span (a lean chain step, few pair boundaries).
//
// Order: externals precede internals in a sorted row (G22) and both are consumed in row
// order with separately rounded mul and add, so x is bit-identical to Alg.1.
// Forward progress: a poller only waits on rows of earlier pairs (earlier CTAs by the start ticket,
// or earlier pairs of its own CTA); a chain warp waits on its own poller.
// UPPER / UNIT (G25): logical row r = physical row n-1-r for upper handles;
// entries are walked earliest-solved first.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

constexpr int kChainPPairs = 2;  // (chain, poller) warp pairs per CTA by default

// per-pair shared memory for RT = 32K rows: f64 c_b, c_d, c_r, c_v, e_ls, s_x, p_nv [RT] |
// i32 f_ji, c_kind, p_j, p_nc [RT], s_rp [RT+1] | u32 ready [K] | i32 win [64]   (16-byte multiple)
__host__ __device__ constexpr int chainp_pair_smem_bytes(int K) {
    return ((8 * 7 * 32 * K + 4 * (4 * 32 * K + 32 * K + 1) + 4 * K + 4 * 64) + 15) / 16 * 16;
}

__device__ __forceinline__ void bar_sync_n(int id, int threads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(threads) : "memory");
}
// the ready mask: the poller's release-OR after the row's partial sum, the chain warp's acquire
// load before reading it (CTA scope, shared memory: no fence on either side)
__device__ __forceinline__ uint32_t ld_acquire_smem_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"((unsigned)__cvta_generic_to_shared(p)) : "memory");
    return v;
}
__device__ __forceinline__ void red_release_cta_or(uint32_t *p, uint32_t v) {
    asm volatile("red.release.cta.shared::cta.or.b32 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(p)), "r"(v) : "memory");
}

template <int PROTO, int K, bool UPPER = false, bool UNIT = false>
__global__ void __launch_bounds__(256) k_solve_chainp(SolveParams p) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint32_t s_blk, s_epoch;
    constexpr int RT = 32 * K;
    const int pairs = blockDim.x >> 6;
    const int pair = threadIdx.x >> 6;
    const bool poller = (threadIdx.x >> 5) & 1;
    const int lane = threadIdx.x & 31;
    const int pt = threadIdx.x & 63;
    if (threadIdx.x == 0) {
        cta_ticket(p, s_blk, s_epoch);
        if (p.bflag && s_blk != kStaleBlk) {  // sptrsv_solve_host: this CTA's b chunks (physical rows)
            const int lr0 = (int)s_blk * pairs * RT, lr1 = min(p.n, lr0 + pairs * RT);
            wait_b_chunks(p, UPPER ? p.n - lr1 : lr0, UPPER ? p.n - lr0 : lr1);
        }
    }
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const int r0 = ((int)s_blk * pairs + pair) * RT;  // the pair's first LOGICAL row
    if (r0 >= p.n) return;                             // both warps of the pair leave together
    const int rows = min(RT, p.n - r0);
    const uint64_t pol = policy_evict_first();
    unsigned char *wsm = smem + (size_t)pair * chainp_pair_smem_bytes(K);
    double *c_b = reinterpret_cast<double *>(wsm);
    double *c_d = c_b + RT, *c_r = c_d + RT, *c_v = c_r + RT, *e_ls = c_v + RT, *s_x = e_ls + RT, *p_nv = s_x + RT;
    int32_t *f_ji = reinterpret_cast<int32_t *>(p_nv + RT);
    int32_t *c_kind = f_ji + RT, *p_j = c_kind + RT, *p_nc = p_j + RT, *s_rp = p_nc + RT;
    uint32_t *ready = reinterpret_cast<uint32_t *>(s_rp + RT + 1);
    int32_t *win = reinterpret_cast<int32_t *>(ready + K);  // the poller's window (row ids)
    const int p0 = UPPER ? p.n - r0 - rows : r0;                    // first physical row of the slice
    auto phys = [&](int lr) { return UPPER ? p.n - 1 - lr : lr; };  // logical row / column -> physical
    auto slot = [&](int t) { return UPPER ? rows - 1 - t : t; };    // pair row t -> s_rp index
    constexpr int dir = UPPER ? -1 : 1;                             // entry walk, earliest-solved first
    auto lcol = [&](int jj) { return UPPER ? p.n - 1 - ld_stream_i32(p.colidx + jj, pol) : ld_stream_i32(p.colidx + jj, pol); };
    auto val_at = [&](int jj) -> double { return ld_stream_f64(p.val + jj, pol); };
    // row t's entries walked from j0 (earliest-solved first) to je (exclusive): the diagonal, or the
    // row's edge for unit forms.  lower: [rs, re-1) ascending, diagonal re-1; upper: (rs, re)
    // descending, diagonal rs.
    auto j0_of = [&](int t) { return UPPER ? s_rp[slot(t) + 1] - 1 : s_rp[slot(t)]; };
    auto je_of = [&](int t) {
        return UPPER ? (UNIT ? s_rp[slot(t)] - 1 : s_rp[slot(t)]) : (UNIT ? s_rp[slot(t) + 1] : s_rp[slot(t) + 1] - 1);
    };
    // ---- setup (both warps, rows strided by 64): rowptr, then every row's constants
    for (int idx = pt; idx <= rows; idx += 64) s_rp[idx] = ld_stream_i32(p.rowptr + p0 + idx, pol);
    for (int idx = pt; idx < K; idx += 64) ready[idx] = 0u;
    bar_sync_n(1 + pair, 64);
    for (int t = pt; t < rows; t += 64) {
        const int j0 = j0_of(t), je = je_of(t);
        // internal entries (logical column >= r0) trail the walk: scan back from its end
        int ji = je, nint = 0, clast = -1;
        while (ji != j0) {
            const int c = lcol(ji - dir);
            if (c < r0) break;
            if (nint == 0) clast = c;
            ji -= dir;
            ++nint;
        }
        const bool k1 = nint == 1 && clast == r0 + t - 1;
        c_kind[t] = nint == 0 ? 0 : k1 ? 1 : 2;
        c_v[t] = k1 ? val_at(ji) : 0.0;
        f_ji[t] = ji;
        Diag dg;
        dg.init(UNIT ? 1.0 : val_at(UPPER ? s_rp[slot(t)] : s_rp[slot(t) + 1] - 1));
        c_d[t] = dg.d;
        c_r[t] = dg.r;
        c_b[t] = ld_b(p, phys(r0 + t), pol);
        e_ls[t] = 0.0;
        p_j[t] = j0;
        if (j0 != ji) {  // an external entry first: the poller's
            p_nc[t] = lcol(j0);
            p_nv[t] = val_at(j0);
        } else {
            p_nc[t] = -1;
            atomicOr(ready + (t >> 5), 1u << (t & 31));
        }
    }
    bar_sync_n(1 + pair, 64);
    uint32_t backoff = p.backoff_min, idle = 0;
    auto watchdog = [&]() -> bool {  // true: abort (a lane-0 check, broadcast)
        uint32_t ab = 0;
        if (lane == 0) {
            if (p.spin_limit && idle >= p.spin_limit) {
                atomicCAS(&p.st->error.v, 0u, kErrTimeout);
                st_relaxed_u32(&p.st->abort.v, 1u);
            }
            ab = ld_relaxed_u32(&p.st->abort.v);
        }
        return __shfl_sync(FULL, ab, 0) != 0;
    };

    if (poller) {
        // ================= POLLER: external entries (logical columns < r0), window of 64 rows
        int lo = 0;  // rows < lo are all handed over
        while (true) {
            __syncwarp();  // p_nc / win written by other lanes
            // the window: the first 64 rows (from lo) that still have an external entry, in row
            // order -- rows behind a blocked one keep consuming (a pair boundary's first row waits
            // for the previous pair's last row while the rows after it consume their norths)
            int cnt = 0;
            bool found = false;
            const int wmax = p.poll_one ? 32 : 64;  // window: 2 rows per lane, or 1 (SPTRSV_OPT_POLL_ONE)
            for (int base = lo; base < rows && cnt < wmax; base += 32) {
                const int t = base + lane;
                const bool pend = t < rows && p_nc[t] >= 0;
                const unsigned m = __ballot_sync(FULL, pend);
                if (!found) {
                    if (m) {
                        lo = base + __ffs(m) - 1;
                        found = true;
                    } else {
                        lo = base + 32;
                    }
                }
                if (pend) {
                    const int r = cnt + __popc(m & ((1u << lane) - 1u));
                    if (r < wmax) win[r] = t;
                }
                cnt += __popc(m);
            }
            if (cnt == 0) break;
            __syncwarp();
            int tt[2], cc[2];
            unsigned long long w0[2], w1[2];
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                tt[u] = lane + 32 * u < min(cnt, wmax) ? win[lane + 32 * u] : -1;
                cc[u] = tt[u] >= 0 ? p_nc[tt[u]] : -1;
                w0[u] = 0;
                w1[u] = 0;
                if (cc[u] >= 0) poll1<PROTO>(p, phys(cc[u]), w0[u], w1[u]);
            }
            bool prog = false;
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                if (cc[u] >= 0 && ready1<PROTO>(w0[u], w1[u], epoch)) {
                    const int t = tt[u];
                    if (p.trace) p.trace[p.n + phys(r0 + t)] = globaltimer_ns();
                    const double ls = __dadd_rn(e_ls[t], __dmul_rn(p_nv[t], value1<PROTO>(p, phys(cc[u]), w0[u], w1[u])));
                    const int j = p_j[t] + dir;
                    e_ls[t] = ls;
                    if (j != f_ji[t]) {  // another external entry: load it (rare: c2-like rows)
                        p_j[t] = j;
                        p_nv[t] = val_at(j);
                        p_nc[t] = lcol(j);
                    } else {  // externals done: hand the row over to the chain warp (release: e_ls first)
                        if (p.trace) p.trace[3 * (size_t)p.n + 3 + phys(r0 + t)] = globaltimer_ns();
                        red_release_cta_or(ready + (t >> 5), 1u << (t & 31));
                        p_nc[t] = -1;
                    }
                    prog = true;
                }
            }
            if (__any_sync(FULL, prog)) {
                backoff = p.backoff_min;
                idle = 0;
                continue;
            }
            if (backoff) nanosleep_ns(backoff);
            backoff = min(max(backoff * 2u, 32u), p.backoff_max);
            if ((++idle & 63u) == 0 && watchdog()) return;
        }
        return;
    }

    // ================= CHAIN: finalize the pair's rows in order
    const bool tracing = p.trace != nullptr;
    int s = 0;          // next row (pair-relative) to finalize
    double xp = 0.0;    // x of row s - 1
    const unsigned long long ep = (unsigned long long)epoch << 32;
    uint32_t wait = 0;
    while (s < rows) {
        // the run of rows s.. whose external entries are all consumed
        int run_end = s;
        {
            int w = s >> 5;
            uint32_t m = ld_acquire_smem_u32(ready + w) >> (s & 31);
            int b = s & 31;
            while (true) {
                const uint32_t z = ~m;
                const int len = z ? __ffs(z) - 1 : 32 - b;
                run_end += len;
                if (z || ++w >= K || run_end >= rows) break;
                m = ld_acquire_smem_u32(ready + w);
                b = 0;
            }
            run_end = min(run_end, rows);
        }
        if (run_end == s) {
            if (wait) nanosleep_ns(wait);
            wait = p.poll_gap ? min(max(wait * 2u, 16u), p.poll_gap) : 0u;
            if ((++idle & 1023u) == 0 && watchdog()) return;
            continue;
        }
        wait = 0;
        idle = 0;
        if (tracing && lane == 0) p.trace[2 * (size_t)p.n + phys(r0 + s)] = globaltimer_ns();  // run start
        const int s0 = s;
        while (s < run_end) {
            // ---- fast loop: rows with no internal entry or exactly the previous row, inside the
            // division guard.  Operands of row t+1 load while row t computes; the only loop-carried
            // value is xp.
            double bv = c_b[s], dv = c_d[s], rv = c_r[s], lv = e_ls[s], vv = c_v[s];
            int kd = c_kind[s];
            int t = s;
            for (; t < run_end; ++t) {
                if (kd == 2) break;
                const int tn = min(t + 1, run_end - 1);
                const double bn = c_b[tn], dn = c_d[tn], rn = c_r[tn], ln = e_ls[tn], vn = c_v[tn];
                const int kn = c_kind[tn];
                const double u = __dadd_rn(lv, __dmul_rn(vv, xp));
                const double a = __dsub_rn(bv, kd ? u : lv);
                double q = a;
                if (!UNIT) {
                    Diag g;
                    g.d = dv;
                    g.r = rv;
                    q = g.cand(a);
                    // the guard (Diag::ok) leaves the loop instead of branching around __ddiv_rn:
                    // no reconvergence point in the loop body
                    if (__builtin_expect(!(Diag::in_range(a) && __double2hiint(rv) != 0 && Diag::exact(a, dv, q)), 0))
                        break;
                }
                s_x[t] = q;  // every lane stores the same value (each lane re-reads its own store)
                if (PROTO == PROTO_FUSED) {
                    unsigned long long bits = (unsigned long long)__double_as_longlong(q);
                    bits = bits == kSentinel ? kCanonNaN : bits;  // same canonicalisation as publish()
                    st_relaxed_v2_u64_if(lane == 0, p.rec + 2 * (size_t)phys(r0 + t), ep | (bits & 0xffffffffull),
                                         ep | (bits >> 32));
                }
                if (tracing) st_u64_if(lane == 0, p.trace + phys(r0 + t), globaltimer_ns());
                xp = q;
                bv = bn, dv = dn, rv = rn, lv = ln, vv = vn, kd = kn;
            }
            s = t;
            if (s >= run_end) break;
            // ---- one general step: a row with several internal entries, or outside the guard
            {
                double a = e_ls[s];
                const int je = je_of(s);
                for (int jj = f_ji[s]; jj != je; jj += dir) {
                    const int c = lcol(jj) - r0;
                    a = __dadd_rn(a, __dmul_rn(val_at(jj), c == s - 1 ? xp : s_x[c]));
                }
                double q;
                if (UNIT) {
                    q = __dsub_rn(c_b[s], a);
                } else {
                    Diag g;
                    g.d = c_d[s];
                    g.r = c_r[s];
                    q = g.div(__dsub_rn(c_b[s], a));
                }
                s_x[s] = q;
                if (PROTO == PROTO_FUSED) {
                    unsigned long long bits = (unsigned long long)__double_as_longlong(q);
                    bits = bits == kSentinel ? kCanonNaN : bits;
                    st_relaxed_v2_u64_if(lane == 0, p.rec + 2 * (size_t)phys(r0 + s), ep | (bits & 0xffffffffull),
                                         ep | (bits >> 32));
                }
                if (tracing) st_u64_if(lane == 0, p.trace + phys(r0 + s), globaltimer_ns());
                xp = q;
                ++s;
            }
        }
        __syncwarp();
        // the run's x (output), coalesced; FLAGS: x stores, one gpu-scope fence, relaxed flags
        for (int t = s0 + lane; t < s; t += 32) {
            p.x[phys(r0 + t)] = s_x[t];
            if (PROTO == PROTO_FLAGS && tracing) p.trace[phys(r0 + t)] = globaltimer_ns();
        }
        if (PROTO == PROTO_FLAGS) {
            fence_acq_rel_gpu();
            for (int t = s0 + lane; t < s; t += 32) st_relaxed_u32(p.flags + phys(r0 + t), epoch);
        }
    }
    if (p.x_host) {  // sptrsv_solve_host: the pair's rows to pinned host memory, coalesced
        __syncwarp();
        for (int t = lane; t < rows; t += 32) p.x_host[phys(r0 + t)] = s_x[t];
    }
}

}  // namespace sptrsv_dev
