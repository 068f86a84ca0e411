// solve_multi.cuh -- multiple right-hand sides (PAPER.md:447:
// "the synchronization-free SpTRSV with multiple right-hand sides [21]").
//
// L X = B for nrhs right-hand sides, row-major: B[i*ldb + r], X[i*ldx + r].
// A row is handled by a GROUP of g lanes (g = nrhs rounded up to a power of two,
// g <= 32): lane r of the group owns component (i, r).  Per component it is the
// thread-level Writing-First loop of Alg.5 -- poll the next
// dependency, consume, solve + publish at the diagonal -- and every (i, r) has
// its own ready word, so the g lanes of a group never synchronise with each
// other: they only share the row's structure and values (same addresses ->
// broadcast loads) and touch contiguous X / record words (coalesced).  The
// dependency hop is paid once per row for all nrhs solves, which is why the
// multi-RHS GFLOPS exceed the single-RHS ones in the latency-bound regimes.
//   PROTO_FUSED: rec[(i*nrhs + r)] = the epoch-tagged record of x_ir;
//   PROTO_FLAGS: flags[i*nrhs + r] with st.release / ld.acquire, x_ir in X.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

struct MultiParams {
    const double *B;
    double *X;
    long long ldb, ldx;
    int nrhs;
    int g;  // lanes per row group (power of two >= nrhs)
};

template <int PROTO>
__global__ void __launch_bounds__(256) k_solve_multi(SolveParams p, MultiParams m) {
    __shared__ uint32_t s_blk, s_epoch;
    const int tid = threadIdx.x;
    const int lane = tid & 31;
    const uint64_t pol = policy_evict_first();
    if (tid == 0) cta_ticket(p, s_blk, s_epoch);
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const int rows_per_cta = blockDim.x / m.g;
    const int i = (int)s_blk * rows_per_cta + tid / m.g;  // row
    const int r = tid % m.g;                               // right-hand side
    const bool act = i < p.n && r < m.nrhs;
    const long long w = (long long)i * m.nrhs + r;  // ready-word index of component (i, r)
    int rs = 0, re = 1;
    double bi = 0.0;
    if (act) {
        rs = ld_stream_i32(p.rowptr + i, pol);
        re = ld_stream_i32(p.rowptr + i + 1, pol);
        bi = m.B[(long long)i * m.ldb + r];
    }
    const int jd = re - 1;
    int j = rs;
    Diag dg;
    dg.init(act ? ld_stream_f64(p.val + jd, pol) : 1.0);
    int nc = (act && j < jd) ? ld_stream_i32(p.colidx + j, pol) : -1;
    double nv = (act && j < jd) ? ld_stream_f64(p.val + j, pol) : 0.0;
    double ls = 0.0;
    bool done = !act;
    uint32_t backoff = p.backoff_min, idle = 0;
    auto poll = [&](int c, unsigned long long &a0, unsigned long long &a1) {
        const long long wc = (long long)c * m.nrhs + r;
        if (PROTO == PROTO_FLAGS) {
            a0 = ld_acquire_u32(p.flags + wc);
            a1 = 0;
        } else {
            ld_relaxed_v2_u64(p.rec + 2 * wc, a0, a1);
        }
    };
    auto value = [&](int c, unsigned long long a0, unsigned long long a1) -> double {
        if (PROTO == PROTO_FLAGS) return ld_relaxed_f64(m.X + (long long)c * m.ldx + r);
        return __longlong_as_double((long long)((a0 & 0xffffffffull) | (a1 << 32)));
    };
    auto publish_ir = [&]() {
        const double xi = dg.div(__dsub_rn(bi, ls));
        if (PROTO == PROTO_FLAGS) {
            m.X[(long long)i * m.ldx + r] = xi;
            st_release_u32(p.flags + w, epoch);
        } else {
            const unsigned long long bits = (unsigned long long)__double_as_longlong(xi);
            const unsigned long long e = (unsigned long long)epoch << 32;
            st_relaxed_v2_u64(p.rec + 2 * w, e | (bits & 0xffffffffull), e | (bits >> 32));
            m.X[(long long)i * m.ldx + r] = xi;
        }
        done = true;
    };
    while (true) {
        bool prog = false;
        if (!done) {
            if (nc < 0) {
                publish_ir();
                prog = true;
            } else {
                unsigned long long a0, a1;
                poll(nc, a0, a1);
                if (ready1<PROTO>(a0, a1, epoch)) {
                    ls = __dadd_rn(ls, __dmul_rn(nv, value(nc, a0, a1)));
                    ++j;
                    nc = j < jd ? ld_stream_i32(p.colidx + j, pol) : -1;
                    nv = j < jd ? ld_stream_f64(p.val + j, pol) : 0.0;
                    prog = true;
                    if (nc < 0) publish_ir();
                }
            }
        }
        if (!__ballot_sync(FULL, !done)) break;
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
                    atomicCAS(&p.st->error.v, 0u, kErrTimeout);
                    st_relaxed_u32(&p.st->abort.v, 1u);
                }
                ab = ld_relaxed_u32(&p.st->abort.v);
            }
            if (__shfl_sync(FULL, ab, 0)) break;
        }
    }
}

}  // namespace sptrsv_dev
