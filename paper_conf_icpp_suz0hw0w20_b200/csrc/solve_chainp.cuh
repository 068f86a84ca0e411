// solve_chainp.cuh -- ENGINE_CHAIN, round 2: in-warp dependency chains with a POLLER warp.
//
// The per-row method is Alg.5's: consume a row's dependencies in row order,
// divide at the diagonal, publish x_i.  Like the round-1 CHAIN engine, the dependencies that fall
// inside a warp's own R = 32K consecutive rows are resolved on chip instead of through a ready
// record, which is what grid wavefronts and pure chains need (row i depends on i-1).  What changes
// is who waits for the EXTERNAL ones (columns before the warp's first row): round 1 let the chain
// warp poll them itself between chain runs, so a pass cost one L2 round trip plus the chain, and a
// north hop of the 2048^2 grid (c3) took 2.3 us (trace: 1.2 us until the value was seen, 1.1 us
// until the row published).  Here every chain warp has a partner warp in the same CTA:
//   POLLER  owns the rows' external entries.  Lane l holds rows l + 32k (k < K); every pass it
//           polls the next external dependency of each pending row (Alg.5 l.8), consumes the
//           ready ones in row order (l.9), and when a row has no external entry left it writes the
//           row's partial sum to shared memory and sets the row's bit in a ready mask.
//   CHAIN   finalizes rows in order: it waits (in shared memory only) for the next row's bit,
//           adds the row's internal entries -- all of them earlier rows of this warp, already
//           final -- divides (Alg.5 l.13) and publishes (l.14-16).  All 32 lanes evaluate the
//           chain redundantly from shared-memory operands, so a step is its dependent fp64
//           operations and nothing else: no shuffle, no vote, no global memory round trip.
// The chain warp never touches a ready record except to publish, and the poller never waits on
// the chain, so a north value reaches the chain one poll after it lands in L2.
//
// Order: externals precede internals in a sorted row (G22) and both are consumed in row
// order with separately rounded mul and add, so x is bit-identical to Alg.1.
// Forward progress: a poller only waits on rows of earlier warps (earlier CTAs by the start
// ticket, or earlier pairs of its own CTA); a chain warp waits on its own poller.
// UPPER / UNIT (G25): logical rows as in the round-1 engine (logical row r =
// physical row n-1-r for upper handles; entries walked earliest-solved first).
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

constexpr int kChainPPairs = 2;  // (chain, poller) warp pairs per CTA by default
constexpr int kChainPEPR = 4;    // staged CSR entries per row (a longer slice reads global memory)

// per-pair shared memory: f64 s_val[RT*EPR] | s_x, f_b, f_d, f_r, e_ls, f_v [RT] ;
// i32 s_col[RT*EPR] | f_ji, f_kind [RT] | s_rp [RT+1] | ready [K]   (16-byte multiple)
__host__ __device__ constexpr int chainp_pair_smem_bytes(int K) {
    return ((8 * (32 * K * kChainPEPR + 6 * 32 * K) + 4 * (32 * K * kChainPEPR + 2 * 32 * K + 32 * K + 1 + K)) + 15) /
           16 * 16;
}

__device__ __forceinline__ void bar_sync_n(int id, int threads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(threads) : "memory");
}
__device__ __forceinline__ uint32_t ld_volatile_smem_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.volatile.shared.u32 %0, [%1];" : "=r"(v) : "r"((unsigned)__cvta_generic_to_shared(p)) : "memory");
    return v;
}

template <int PROTO, int K, bool UPPER = false, bool UNIT = false>
__global__ void __launch_bounds__(256) k_solve_chainp(SolveParams p) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint32_t s_blk, s_epoch;
    constexpr int RT = 32 * K;
    constexpr int ECAP = RT * kChainPEPR;
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
    double *s_val = reinterpret_cast<double *>(wsm);
    double *s_x = s_val + ECAP;
    double *f_b = s_x + RT, *f_d = f_b + RT, *f_r = f_d + RT, *e_ls = f_r + RT, *f_v = e_ls + RT;
    int32_t *s_col = reinterpret_cast<int32_t *>(f_v + RT);
    int32_t *f_ji = s_col + ECAP, *f_kind = f_ji + RT;
    int32_t *s_rp = f_kind + RT;
    uint32_t *ready = reinterpret_cast<uint32_t *>(s_rp + RT + 1);
    const int p0 = UPPER ? p.n - r0 - rows : r0;                    // first physical row of the slice
    auto phys = [&](int lr) { return UPPER ? p.n - 1 - lr : lr; };  // logical row / column -> physical
    auto slot = [&](int t) { return UPPER ? rows - 1 - t : t; };    // warp row t -> s_rp index
    constexpr int dir = UPPER ? -1 : 1;                             // entry walk, earliest-solved first
    // ---- stage rowptr, b, then the pair's contiguous CSR slice (coalesced, both warps)
    for (int idx = pt; idx <= rows; idx += 64) s_rp[idx] = ld_stream_i32(p.rowptr + p0 + idx, pol);
    for (int idx = pt; idx < rows; idx += 64) f_b[idx] = ld_b(p, phys(r0 + idx), pol);
    if (pt < K) ready[pt] = 0u;
    bar_sync_n(1 + pair, 64);
    const int base = s_rp[0];
    const int len = s_rp[rows] - base;
    const bool staged = len <= ECAP;  // pair-uniform
    if (staged) {
        for (int e = pt; e < len; e += 64) {
            s_col[e] = ld_stream_i32(p.colidx + base + e, pol);
            s_val[e] = ld_stream_f64(p.val + base + e, pol);
        }
    }
    bar_sync_n(1 + pair, 64);
    auto col_at = [&](int jj) -> int { return staged ? s_col[jj - base] : ld_stream_i32(p.colidx + jj, pol); };
    auto val_at = [&](int jj) -> double { return staged ? s_val[jj - base] : ld_stream_f64(p.val + jj, pol); };
    auto lcol = [&](int jj) { return UPPER ? p.n - 1 - col_at(jj) : col_at(jj); };
    // row t: entries walked from j0 (earliest-solved first) up to je (exclusive): the diagonal, or the
    // row's edge for unit forms.  lower: [rs, re-1) ascending, diagonal re-1; upper: (rs, re)
    // descending, diagonal rs.
    auto j0_of = [&](int t) { return UPPER ? s_rp[slot(t) + 1] - 1 : s_rp[slot(t)]; };
    auto je_of = [&](int t) {
        return UPPER ? (UNIT ? s_rp[slot(t)] - 1 : s_rp[slot(t)]) : (UNIT ? s_rp[slot(t) + 1] : s_rp[slot(t) + 1] - 1);
    };
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
        // ================= POLLER: external entries (columns < r0) of the pair's rows
        int j[K], nc[K];
        double nv[K], ls[K];
        unsigned pend = 0;  // bit k: row lane + 32k still has external entries
        // a row whose external entries are consumed: its partial sum to the chain warp
        auto hand_over = [&](int t, double v) {
            e_ls[t] = v;
            __threadfence_block();
            atomicOr(ready + (t >> 5), 1u << (t & 31));
        };
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const int t = lane + 32 * k;
            j[k] = 0;
            nc[k] = -1;
            nv[k] = 0.0;
            ls[k] = 0.0;
            if (t < rows) {
                j[k] = j0_of(t);
                const int c = j[k] != je_of(t) ? lcol(j[k]) : -1;
                if (c >= 0 && c < r0) {
                    nc[k] = c;
                    nv[k] = val_at(j[k]);
                    pend |= 1u << k;
                } else {
                    hand_over(t, 0.0);
                }
            }
        }
        while (__any_sync(FULL, pend != 0)) {
            unsigned long long w0[K], w1[K];
#pragma unroll
            for (int k = 0; k < K; ++k) {
                w0[k] = 0;
                w1[k] = 0;
                if (pend >> k & 1u) poll1<PROTO>(p, phys(nc[k]), w0[k], w1[k]);
            }
            bool prog = false;
#pragma unroll
            for (int k = 0; k < K; ++k) {
                if ((pend >> k & 1u) && ready1<PROTO>(w0[k], w1[k], epoch)) {
                    const int t = lane + 32 * k;
                    if (p.trace) p.trace[p.n + phys(r0 + t)] = globaltimer_ns();
                    ls[k] = __dadd_rn(ls[k], __dmul_rn(nv[k], value1<PROTO>(p, phys(nc[k]), w0[k], w1[k])));
                    j[k] += dir;
                    const int c = j[k] != je_of(t) ? lcol(j[k]) : -1;
                    if (c >= 0 && c < r0) {
                        nc[k] = c;
                        nv[k] = val_at(j[k]);
                    } else {
                        pend &= ~(1u << k);
                        hand_over(t, ls[k]);
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
    // per-row constants (lane-parallel): divisor, its reciprocal, the first internal entry and
    // the internal part's shape: kind 0 = none, 1 = exactly the previous row, 2 = general
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const int t = lane + 32 * k;
        if (t < rows) {
            const int je = je_of(t);
            int jj = j0_of(t);
            while (jj != je && lcol(jj) < r0) jj += dir;  // skip the external prefix
            const int nint = (je - jj) * dir;
            int kind = 2;
            double v1 = 0.0;
            if (nint == 0) {
                kind = 0;
            } else if (nint == 1 && lcol(jj) == r0 + t - 1) {
                kind = 1;
                v1 = val_at(jj);
            }
            Diag dg;
            dg.init(UNIT ? 1.0 : val_at(UPPER ? s_rp[slot(t)] : s_rp[slot(t) + 1] - 1));
            f_d[t] = dg.d;
            f_r[t] = dg.r;
            f_ji[t] = jj;
            f_kind[t] = kind;
            f_v[t] = v1;
        }
    }
    __syncwarp();
    const bool tracing = p.trace != nullptr;
    int s = 0;          // next row (pair-relative) to finalize
    double xp = 0.0;    // x of row s - 1
    while (s < rows) {
        // the run of rows s.. whose external entries are all consumed
        unsigned long long m = ld_volatile_smem_u32(ready);
        if (K == 2) m |= (unsigned long long)ld_volatile_smem_u32(ready + 1) << 32;
        const unsigned long long nm = ~m >> s;
        const int run_end = min(rows, nm ? s + __ffsll((long long)nm) - 1 : 64);
        if (run_end == s) {
            if (p.poll_gap) nanosleep_ns(p.poll_gap);
            if ((++idle & 1023u) == 0 && watchdog()) return;
            continue;
        }
        idle = 0;
        __threadfence_block();  // e_ls of the run was written before its ready bits
        // operands of row t are loaded one row ahead, off the dependency chain
        double bv = f_b[s], dv = f_d[s], rv = f_r[s], lv = e_ls[s], vv = f_v[s];
        int kd = f_kind[s];
        for (int t = s; t < run_end; ++t) {
            const int tn = min(t + 1, run_end - 1);
            const double bn = f_b[tn], dn = f_d[tn], rn = f_r[tn], ln = e_ls[tn], vn = f_v[tn];
            const int kn = f_kind[tn];
            double a = lv;
            if (kd == 1) {
                a = __dadd_rn(a, __dmul_rn(vv, xp));
            } else if (kd == 2) {  // general internal part, in row order (every column < t is final)
                const int je = je_of(t);
                for (int jj = f_ji[t]; jj != je; jj += dir) {
                    const int c = lcol(jj) - r0;
                    a = __dadd_rn(a, __dmul_rn(val_at(jj), c == t - 1 ? xp : s_x[c]));
                }
            }
            double q;
            if (UNIT) {
                q = __dsub_rn(bv, a);
            } else {
                Diag g;
                g.d = dv;
                g.r = rv;
                q = g.div(__dsub_rn(bv, a));
            }
            s_x[t] = q;  // every lane stores the same value (each lane re-reads its own store)
            if (PROTO == PROTO_FUSED) {
                unsigned long long bits = (unsigned long long)__double_as_longlong(q);
                bits = bits == kSentinel ? kCanonNaN : bits;  // same canonicalisation as publish()
                const unsigned long long e = (unsigned long long)epoch << 32;
                st_relaxed_v2_u64_if(lane == 0, p.rec + 2 * (size_t)phys(r0 + t), e | (bits & 0xffffffffull),
                                     e | (bits >> 32));
                if (tracing) st_u64_if(lane == 0, p.trace + phys(r0 + t), globaltimer_ns());
            }
            xp = q;
            bv = bn, dv = dn, rv = rn, lv = ln, vv = vn, kd = kn;
        }
        __syncwarp();
        // the run's x (output), coalesced; FLAGS: x stores, one gpu-scope fence, relaxed flags
        for (int t = s + lane; t < run_end; t += 32) {
            p.x[phys(r0 + t)] = s_x[t];
            if (PROTO == PROTO_FLAGS && tracing) p.trace[phys(r0 + t)] = globaltimer_ns();
        }
        if (PROTO == PROTO_FLAGS) {
            fence_acq_rel_gpu();
            for (int t = s + lane; t < run_end; t += 32) st_relaxed_u32(p.flags + phys(r0 + t), epoch);
        }
        s = run_end;
    }
    if (p.x_host) {  // sptrsv_solve_host: the pair's rows to pinned host memory, coalesced
        for (int t = lane; t < rows; t += 32) p.x_host[phys(r0 + t)] = s_x[t];
    }
}

}  // namespace sptrsv_dev
