// solve_small.cuh -- ENGINE_SMALL: a whole small system solved by ONE CTA out of shared memory.
//
// Alg.5 with every ready signal on chip.  For a system whose CSR arrays, b and x
// fit in one SM's shared memory (c1: 1,000 rows, 3,994 entries = 76 KB), the multi-CTA engines pay
// an L2 round trip per dependency hop (~0.6-0.8 us measured per level of c1, 34 levels) and a
// dependent rowptr -> entries load chain per CTA.  Here:
//   1. the CTA streams rowptr, colidx and val into shared memory by TMA bulk copies (one thread
//      issues them; nnz is known on the host, so no copy waits for another) and b by independent
//      loads (measured: per-thread load loops put 7.7 us of serialized latency before the first
//      row with 256 threads on c1, the bulk copies ~1 us), fills the shared copy of x
//      with the sentinel -- the paper's get_value flags (Alg.5 l.2) are the x words themselves
//      (value-as-flag, as in the ONE-SHOT engine's in-CTA copy) -- and takes each row's
//      reciprocal diagonal off the critical path;
//   2. thread t owns logical rows t, t + T, t + 2T, ... (T threads) and runs Writing-First on its
//      current row, one PASS at a time: poll the next two dependencies' x words, consume the ready
//      prefix in row order (left_sum += L_ij * x_j, separately rounded, Alg.1 l.3-4), and when the
//      prefix reaches the diagonal (Alg.5 l.12-16) store x_i = the Markstein candidate of
//      (b_i - left_sum) / L_ii and move to the thread's next row.  The pass is BRANCH-FREE (every
//      step predicated or selected): on sm_100a a pass whose lanes diverge and re-converge costs
//      ~265 cycles against ~96 for the predicated one (tools/micro/smallstep.cu), and a dependency
//      hop inside a warp is one pass.  The lowest unsolved row's thread is always on that row (its
//      earlier rows are lower, hence solved), so the sweep always progresses -- no tickets;
//   3. the candidates' remainder proofs (Diag::exact) run in one pass after the sweep; a failure
//      (a quotient within ~2^-53 ulp of a rounding midpoint, or an operand outside the guarded
//      range) re-runs the sweep with the verified division of solve.cuh (Diag::div), so x is
//      always the correctly rounded result;
//   4. x is written to global memory with coalesced stores (in the same pass as the proofs).
// Triangular forms (f4): UPPER takes logical row r as row n-1-r with its off-diagonals in
// DESCENDING column order (G25); UNIT has no stored diagonal (x_i = b_i - left_sum).
// No epoch, no flags and no records: nothing persists between solves, so a solve is one launch and
// graph replays are correct; a replay of a graph captured under another configuration still reports
// SPTRSV_ERR_STALE_LAUNCH (generation check on the start-ticket word), like every other engine.
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "solve.cuh"

namespace sptrsv_dev {

constexpr int kSmallCtaMax = 1024;

__host__ __device__ inline size_t small_up16(size_t v) { return (v + 15) & ~(size_t)15; }

// Shared-memory bytes of a system: x words, b, 1 / L_ii (8 B per row), rowptr (4 B per row + 1),
// val (8 B per entry) and colidx (4 B per entry), each array 16-byte aligned (and at least 16 B),
// plus 16 B of slack per streamed array (its shared copy takes the global array's offset mod 16, so
// the bulk copy's interior is 16-byte aligned on both sides).
__host__ __device__ inline size_t small_smem_bytes(long long n, long long nnz) {
    const size_t z = nnz > 0 ? (size_t)nnz : 1;
    return small_up16(8 * (size_t)n) * 3 + small_up16(8 * z) + small_up16(4 * (size_t)(n + 1)) + small_up16(4 * z) +
           4 * 16;
}

__device__ __forceinline__ void st_volatile_smem_u64_if(unsigned addr, unsigned long long v, bool pred) {
    asm volatile("{.reg .pred q; setp.ne.u32 q, %2, 0; @q st.volatile.shared.u64 [%0], %1;}" ::"r"(addr), "l"(v),
                 "r"((unsigned)pred)
                 : "memory");
}

// One array into shared memory: the 16-byte aligned interior by a TMA bulk copy (thread 0, counted
// on the mbarrier `bar`), the < 16-byte head and tail by threads 1..8 as 4-byte words.  `dst` has
// the same offset mod 16 as `src`.  Returns the bytes the bulk copy will complete on the barrier.
__device__ __forceinline__ uint32_t small_stream_in(void *dst, const void *src, size_t bytes, unsigned bar, int tid) {
    const uintptr_t g = (uintptr_t)src;
    const uintptr_t a = (g + 15) & ~(uintptr_t)15, e = (g + bytes) & ~(uintptr_t)15;
    const size_t head = a < g + bytes ? a - g : bytes;  // all of it when there is no aligned interior
    const size_t mid = a < e ? e - a : 0;
    const size_t tail = bytes - head - mid;
    if (tid == 0 && mid) {
        const unsigned d = (unsigned)__cvta_generic_to_shared((char *)dst + head);
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d),
                     "l"(a), "r"((unsigned)mid), "r"(bar)
                     : "memory");
    }
    // head and tail: at most 3 + 3 words (every array here is 4-byte aligned, 4-byte multiples)
    const int w = tid - 1;
    if (w >= 0 && w < 8) {
        const size_t nh = head / 4, nt = tail / 4;
        if ((size_t)w < nh) ((uint32_t *)dst)[w] = __ldg((const uint32_t *)src + w);
        else if ((size_t)w - nh < nt) {
            const size_t k = (head + mid) / 4 + (w - nh);
            ((uint32_t *)dst)[k] = __ldg((const uint32_t *)src + k);
        }
    }
    return (uint32_t)mid;
}

template <bool UPPER, bool UNIT>
__global__ void __launch_bounds__(kSmallCtaMax, 1) k_solve_small(SolveParams p) {
    extern __shared__ __align__(16) unsigned char sm[];
    __shared__ uint32_t s_stale;
    const int n = p.n;
    const long long nnz = p.nnz;
    const size_t z = nnz > 0 ? (size_t)nnz : 1;
    const int T = (int)blockDim.x;
    const int tid = threadIdx.x;
    __shared__ __align__(8) unsigned long long s_bar;
    // layout: x words, b, 1 / L_ii, then val, rowptr, colidx -- each streamed array placed at its
    // global address's offset mod 16 (small_stream_in)
    auto mis = [](const void *q) { return (size_t)((uintptr_t)q & 15); };
    unsigned long long *xs = (unsigned long long *)sm;
    double *bs = (double *)(sm + small_up16(8 * (size_t)n));
    double *rcs = (double *)(sm + 2 * small_up16(8 * (size_t)n));
    unsigned char *tail0 = sm + 3 * small_up16(8 * (size_t)n);
    double *vs = (double *)(tail0 + mis(p.val));
    unsigned char *tail1 = tail0 + small_up16(8 * z) + 16;
    int32_t *rp = (int32_t *)(tail1 + mis(p.rowptr));
    unsigned char *tail2 = tail1 + small_up16(4 * (size_t)(n + 1)) + 16;
    int32_t *cs = (int32_t *)(tail2 + mis(p.colidx));
    const uint64_t pol = policy_evict_first();
    const unsigned bar = (unsigned)__cvta_generic_to_shared(&s_bar);
    if (tid == 0) {
        if (p.trace) p.trace[3 * (size_t)n] = globaltimer_ns();
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    __syncthreads();
    // ---- 1. the system into shared memory: TMA bulk copies of val, rowptr and colidx (one thread
    // issues them, the copy engine streams them), b too when it is 16-byte aligned device memory (else
    // by the threads: under sptrsv_solve_host it lives in mapped host memory), x words set to the sentinel
    uint32_t tx = 0;
    if (nnz > 0) {
        tx += small_stream_in(vs, p.val, 8 * (size_t)nnz, bar, tid);
        tx += small_stream_in(cs, p.colidx, 4 * (size_t)nnz, bar, tid);
    }
    tx += small_stream_in(rp, p.rowptr, 4 * (size_t)(n + 1), bar, tid);
    const bool b_bulk = p.x_host == nullptr && ((uintptr_t)p.b & 15) == 0;  // b in device memory, aligned
    if (b_bulk) tx += small_stream_in(bs, p.b, 8 * (size_t)n, bar, tid);
    if (tid == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(tx) : "memory");
    if (!b_bulk) {
        for (int k0 = tid; k0 < n; k0 += 4 * T) {  // four independent loads in flight per thread
            double v[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) v[u] = k0 + u * T < n ? ld_stream_f64(p.b + k0 + u * T, pol) : 0.0;
#pragma unroll
            for (int u = 0; u < 4; ++u)
                if (k0 + u * T < n) bs[k0 + u * T] = v[u];
        }
    }
    for (int k = tid; k < n; k += T) xs[k] = kSentinel;
    if (tid == (T > 32 ? 32 : 0)) {
        // a graph captured under an earlier configuration (sptrsv.cu reset_state bumps gen); checked by
        // a thread of the second warp while the copies stream
        const unsigned long long tk = ld_relaxed_u64(&p.st->tk.v);
        s_stale = (uint32_t)(tk >> kGenShift) != p.gen;
        if (s_stale) {
            atomicCAS(&p.st->error.v, 0u, kErrStale);
            st_relaxed_u32(&p.st->abort.v, 1u);
        }
    }
    if (nnz == 0 && tid == 0) {  // (UNIT, no entries: the passes read one dummy entry)
        cs[0] = 0;
        vs[0] = 0.0;
    }
    asm volatile("{.reg .pred p; WAIT_%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0; @!p bra WAIT_%=;}" ::"r"(
                     bar)
                 : "memory");
    __syncthreads();
    if (s_stale) return;
    if (!UNIT) {  // 1 / L_ii, 0 outside the guarded range (Diag::init)
        for (int k = tid; k < n; k += T) {
            const double d = vs[UPPER ? rp[k] : rp[k + 1] - 1];
            rcs[k] = Diag::in_range(d) ? __drcp_rn(d) : 0.0;
        }
        __syncthreads();
    }
    const unsigned xs_s = (unsigned)__cvta_generic_to_shared(xs);
    constexpr int dir = UPPER ? -1 : 1;
    // ---- 2. the fast sweep: branch-free passes
    {
        int r = tid;
        bool act = r < n;
        int i, j, e;  // row, next entry, end of the off-diagonals (direction dir)
        double ls, bi, d, rc;
        auto load_row = [&](int rr) {  // rr < n (callers clamp)
            i = UPPER ? n - 1 - rr : rr;
            const int rs = rp[i], re = rp[i + 1];
            j = UPPER ? re - 1 : rs;
            e = UPPER ? (UNIT ? rs : rs + 1) - 1 : (UNIT ? re : re - 1);
            bi = bs[i];
            d = UNIT ? 1.0 : vs[UPPER ? rs : re - 1];
            rc = UNIT ? 1.0 : rcs[i];
            ls = 0.0;
        };
        // (lanes without a row keep running the passes on a clamped dummy row 0, their loads and
        // results discarded: compute-sanitizer racecheck reports those reads against row 0's
        // stores, and the value-as-flag polls against the publishes -- both by design)
        load_row(act ? r : 0);
        uint32_t idle_ns = 0;
        while (__any_sync(FULL, act)) {
            const bool h0 = act && j != e;
            const bool h1 = h0 && j + dir != e;
            const int j0 = h0 ? j : 0, j1 = h1 ? j + dir : 0;
            const int c0 = cs[j0], c1 = cs[j1];
            const unsigned long long v0 = ld_volatile_smem_u64_at(xs_s + 8u * (unsigned)(h0 ? c0 : 0));
            const unsigned long long v1 = ld_volatile_smem_u64_at(xs_s + 8u * (unsigned)(h1 ? c1 : 0));
            const bool r0 = h0 && v0 != kSentinel;
            const bool r1 = r0 && h1 && v1 != kSentinel;
            const double l1 = __dadd_rn(ls, __dmul_rn(vs[j0], __longlong_as_double((long long)v0)));
            const double l2 = __dadd_rn(l1, __dmul_rn(vs[j1], __longlong_as_double((long long)v1)));
            ls = r1 ? l2 : r0 ? l1 : ls;
            j += r1 ? 2 * dir : r0 ? dir : 0;
            const bool fin = act && j == e;
            const double a = __dsub_rn(bi, ls);
            double xi = a;
            if (!UNIT) {  // the Markstein candidate; its proof is deferred to step 3
                const double q0 = __dmul_rn(a, rc);
                xi = __fma_rn(__fma_rn(-q0, d, a), rc, q0);
            }
            unsigned long long bits = (unsigned long long)__double_as_longlong(xi);
            bits = bits == kSentinel ? kCanonNaN : bits;  // never publish the sentinel (NaN payload only)
            st_volatile_smem_u64_if(xs_s + 8u * (unsigned)i, bits, fin);
            if (!UNIT && fin) bs[i] = a;  // b_i is dead: keep a for the proof
            if (p.trace && fin) p.trace[i] = globaltimer_ns();
            r += fin ? T : 0;
            act = r < n;
            if (!__any_sync(FULL, r0 || fin)) {  // no progress: yield the issue slots for a while
                if (idle_ns) nanosleep_ns(idle_ns);
                idle_ns = min(max(idle_ns * 2u, p.backoff_min), p.backoff_max);
                continue;
            }
            idle_ns = 0;
            if (__any_sync(FULL, fin)) {  // warp-uniform: some lane moves on to its next row
                const int i_old = i, j_old = j, e_old = e;
                const double ls_old = ls, bi_old = bi, d_old = d, rc_old = rc;
                load_row(act ? r : 0);
                if (!fin) {
                    i = i_old, j = j_old, e = e_old;
                    ls = ls_old, bi = bi_old, d = d_old, rc = rc_old;
                }
            }
        }
    }
    __syncthreads();
    if (!UNIT) {
        // ---- 3. the deferred proof: every candidate must be RN(a / L_ii) (Diag::exact, inside the
        // guarded range; a = 0 gives the exact signed zero); a failure re-runs the sweep with the
        // verified division, b reloaded and x back to the sentinel
        // (fused with step 4: x goes out with its proof; a re-run writes it again)
        bool bad = p.chain_div == 2;  // test hook (SPTRSV_OPT_CHAIN_DIV = 2): every proof fails
        for (int k = tid; k < n; k += T) {
            const int rs = rp[k], re = rp[k + 1];
            const double d = vs[UPPER ? rs : re - 1], a = bs[k];
            const double q = __longlong_as_double((long long)xs[k]);
            const bool ok = Diag::in_range(d) && (a == 0.0 || (Diag::in_range(a) && Diag::exact(a, d, q)));
            bad |= !ok;
            p.x[k] = q;
            if (p.x_host) p.x_host[k] = q;
        }
        if (__syncthreads_or(bad)) {
            for (int k = tid; k < n; k += T) {
                bs[k] = ld_stream_f64(p.b + k, pol);
                xs[k] = kSentinel;
            }
            __syncthreads();
            int r = tid, i = 0, j = 0, e = 0;
            double ls = 0.0;
            Diag dg;
            auto load_row = [&]() {
                i = UPPER ? n - 1 - r : r;
                const int rs = rp[i], re = rp[i + 1];
                j = UPPER ? re - 1 : rs;
                e = UPPER ? rs : re - 1;
                dg.init(vs[UPPER ? rs : re - 1]);
                ls = 0.0;
            };
            bool act = r < n;
            if (act) load_row();
            while (__any_sync(FULL, act)) {
                if (!act) continue;
                while (j != e) {  // the ready prefix (finite: at most the row's length)
                    const unsigned long long v = ld_volatile_smem_u64_at(xs_s + 8u * (unsigned)cs[j]);
                    if (v == kSentinel) break;
                    ls = __dadd_rn(ls, __dmul_rn(vs[j], __longlong_as_double((long long)v)));
                    j += dir;
                }
                if (j != e) continue;
                unsigned long long bits = (unsigned long long)__double_as_longlong(dg.div(__dsub_rn(bs[i], ls)));
                if (bits == kSentinel) bits = kCanonNaN;
                asm volatile("st.volatile.shared.u64 [%0], %1;" ::"r"(xs_s + 8u * (unsigned)i), "l"(bits) : "memory");
                r += T;
                act = r < n;
                if (act) load_row();
            }
            __syncthreads();
            for (int k = tid; k < n; k += T) {
                const double xv = __longlong_as_double((long long)xs[k]);
                p.x[k] = xv;
                if (p.x_host) p.x_host[k] = xv;
            }
        }
    } else {
        // ---- 4. x to global memory (and to pinned host memory for sptrsv_solve_host)
        for (int k = tid; k < n; k += T) {
            const double xv = __longlong_as_double((long long)xs[k]);
            p.x[k] = xv;
            if (p.x_host) p.x_host[k] = xv;
        }
    }
    if (p.trace && tid == 0) p.trace[3 * (size_t)n + 1] = globaltimer_ns();
}

}  // namespace sptrsv_dev
