// solve_grid.cuh -- ENGINE_GRID: wavefront bands for stencil-shaped lower factors.
//
// The same per-row method as every engine -- Alg.5's row: the off-diagonals
// consumed in column order with separately rounded mul / add, the division at the diagonal, the
// publish -- mapped onto the shape of the paper's low-parallelism regime (Table 6, PAPER.md:421-437:
// small beta = n / levels): lower factors of structured grids, where row r = y*m + x (line y,
// column x) depends on its west neighbour r-1 and its north neighbour r-m (5-point stencil), plus at
// most one far row (7-point: the plane below).  CHAIN walks such a matrix in row order, so each grid
// line waits for the line above through the global protocol (c3, 2048^2: ~2.4 us per line).
//
// GRID cuts the matrix into BANDS of 32 columns: band k = columns [32k, 32k+32) of every line.  Lane
// l of band k's warp owns column x = 32k + l and walks the lines with a skew of one step per lane
// (step s: lane l solves line y = s - l).  Then
//   north (r - m)  = the lane's own result of the previous step       (a register)
//   west  (r - 1)  = lane l-1's result of the previous step           (one __shfl_up_sync)
//   lane 0's west  = band k-1's lane 31, through the global protocol, polled by the band's RING warp
//                    32 lines per round trip and handed over in shared memory
//   a far entry    = the global protocol, polled by the producer warp that prepares the row
// so a step costs one shuffle and the row's dependent fp64 operations, and band k waits on band k-1
// through lane 0 only: one global hop per 32 columns instead of one per line.  The critical path is
// the grid's wavefront, lines + 32 * bands steps, plus one hop per band.  Measured (c3, 2048^2 grid,
// B200): 0.87 ms against CHAIN's 5.10 ms; see DESIGN.md section 6 for the design steps and what each
// one bought (a per-step poll held in lane registers cost a round trip per step through the warp's
// scoreboard -- hence the ring warp).
//
// Eligibility (k_grid_check, every row, for the m k_grid_probe proposes): each off-diagonal is the
// west neighbour (c = r - 1 with x >= 1), the north neighbour (c = r - m), or a far entry c < r - m
// that lies in an earlier band, or in the same band at an earlier step; at most one far entry.
// That is exactly when no step waits on a later step of its own band or on a later band (forward
// progress: bands take the CTA start ticket, so band k only waits on bands started before it).
// Accumulation far -> north -> west is column order with separately rounded mul and add, as Alg.1
// (PAPER.md:82-92): x is bit-identical to the oracle.  Division: Diag (solve.cuh) -- the Markstein
// candidate, proven by its remainder either in the loop (SAFE) or off the chain with the failure
// reported as SPTRSV_ERR_INEXACT (the CHAIN contract, SPTRSV_OPT_CHAIN_DIV).
#pragma once
#include <cstdint>

#include "ptx.cuh"
#include "setup.cuh"
#include "solve.cuh"

namespace sptrsv_dev {


// ---------------------------------------------------------------- analyse: is the matrix a grid?

// The triangular forms (G25) in LOGICAL rows: an upper handle solves logical row
// r = n-1-i (physical row i), so its dependencies are logical columns n-1-c < r and the whole analysis
// (and the engine) runs on the logical lower matrix; the off-diagonals of physical row [s, e):
//   lower: [s, e-1) (diagonal last), unit lower: [s, e); upper: [s+1, e) (diagonal first), unit upper: [s, e)
// and in logical column order they run ascending (lower) or descending (upper).
struct GridForm {
    bool up, unit;
    int32_t n;
    __device__ int logical(int i) const { return up ? n - 1 - i : i; }
    __device__ void offdiag(int s, int e, int &lo, int &hi) const {
        lo = (up && !unit) ? s + 1 : s;
        hi = (!up && !unit) ? e - 1 : e;
    }
    // position of the t-th off-diagonal counted from the logically LAST one (t = 0: nearest dependency)
    __device__ int from_last(int lo, int hi, int t) const { return up ? lo + t : hi - 1 - t; }
};

// One warp proposes the line length m: each lane samples one logical row and takes the distance to its
// nearest off-diagonal that is not the previous row (the north neighbour of a grid row); the most
// frequent candidate (>= 2 votes) wins.  Upper handles need n to be a multiple of m (whole lines).
__global__ void k_grid_probe(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ colidx, int32_t n,
                             AnalyseOut *out, int tri) {
    const int lane = threadIdx.x;
    const GridForm f{(tri & 1) != 0, (tri & 2) != 0, n};
    int cand = 0;
    const bool valid = out->status == ~0ull && n >= 2;
    if (valid) {
        const int rl = (int)((long long)(lane + 1) * n / 33);
        const int i = f.logical(rl);
        int lo, hi;
        f.offdiag(rowptr[i], rowptr[i + 1], lo, hi);
        int t = 0;
        if (hi > lo && f.logical(colidx[f.from_last(lo, hi, 0)]) == rl - 1) t = 1;
        if (hi - lo > t) cand = rl - f.logical(colidx[f.from_last(lo, hi, t)]);
    }
    const unsigned same = __match_any_sync(0xffffffffu, cand);
    const unsigned cnt = cand > 1 ? (unsigned)__popc(same) : 0u;
    unsigned long long key = ((unsigned long long)cnt << 32) | (unsigned)cand;
    for (int off = 16; off; off >>= 1) {
        const unsigned long long o = __shfl_xor_sync(0xffffffffu, key, off);
        key = o > key ? o : key;
    }
    if (lane == 0) {
        int m = (valid && (key >> 32) >= 2) ? (int)(key & 0xffffffffu) : 0;
        if (f.up && m > 0 && n % m != 0) m = 0;
        out->grid_m = m;
    }
}

// Every row against the m of k_grid_probe: violations of the band order (see the header), fast
// entries (north / west) and far entries, in logical rows and columns.
__global__ void __launch_bounds__(256) k_grid_check(const int32_t *__restrict__ rowptr,
                                                    const int32_t *__restrict__ colidx, int32_t n, AnalyseOut *out,
                                                    int tri) {
    const int m = out->grid_m;
    if (m < 2 || out->status != ~0ull) return;
    const GridForm f{(tri & 1) != 0, (tri & 2) != 0, n};
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    unsigned viol = 0, fast = 0, far = 0;
    if (i < n) {
        const int r = f.logical(i);
        const int y = r / m, x = r - y * m, k = x >> 5, l = x & 31;
        int lo, hi;
        f.offdiag(rowptr[i], rowptr[i + 1], lo, hi);
        for (int j = lo; j < hi; ++j) {
            const int c = f.logical(colidx[j]);
            if ((c == r - 1 && x >= 1) || c == r - m) {
                ++fast;
            } else if (c < r - m) {
                const int y2 = c / m, x2 = c - y2 * m, k2 = x2 >> 5, l2 = x2 & 31;
                if (!(k2 < k || (k2 == k && y2 + l2 < y + l))) viol = 1;
                ++far;
            } else {
                viol = 1;  // between the north and the west neighbour, or r-1 across a line start
            }
        }
        if (far > 1) viol = 1;
    }
    for (int off = 16; off; off >>= 1) {
        viol += __shfl_xor_sync(0xffffffffu, viol, off);
        fast += __shfl_xor_sync(0xffffffffu, fast, off);
        far += __shfl_xor_sync(0xffffffffu, far, off);
    }
    if ((threadIdx.x & 31) == 0) {
        if (viol) atomicAdd(&out->grid_viol, (int)viol);
        if (fast) atomicAdd((unsigned long long *)&out->grid_fast, (unsigned long long)fast);
        if (far) atomicAdd((unsigned long long *)&out->grid_far, (unsigned long long)far);
    }
}

// ---------------------------------------------------------------- the solve
//
// One band per CTA of six warps: warp 0, the CONSUMER, runs the band's chain (the skewed steps
// above) and nothing else; warps 1..kGridProd, the PRODUCERS, keep it fed (the last warp is the RING):
//   - raw CSR staging: the rows of one line of a band are contiguous, so rowptr / b / entries of a
//     line are copied into a shared-memory ring (kGridRaw lines) by cp.async, coalesced, kGridA1 /
//     kGridA2 blocks before they are needed;
//   - classification: each staged row becomes a DESCRIPTOR (ls0 = its far entry's product already
//     summed when the far row was published, north / west coefficients, b, d, RN(1/d), flags) in a
//     second ring (kGridDesc lines).
// The CTA meets at a barrier every kGridBlk consumer steps: block b runs steps [B*b, B*b + B) and
// produces the descriptors of lines [B*b + B + 1, B*b + 2B] (B = kGridBlk), so the consumer always
// finds the next B + 1 lines ready and its step is one shuffle, the row's dependent fp64 operations,
// two stores and one-step-ahead shared-memory loads.
constexpr int kGridProd = 4;              // producer warps
constexpr int kGridBlk = 2 * kGridProd;   // consumer steps per block (each producer: 2 lines per block)
constexpr int kGridDesc = 48;             // descriptor ring (lines): line y is read until step y + 30
constexpr int kGridRaw = 64;              // raw CSR ring (lines)
constexpr int kGridA1 = 6;                // rowptr / b staged this many blocks before production
constexpr int kGridA2 = 3;                // entries staged this many blocks before production
constexpr int kGridWarps = 2 + kGridProd;  // consumer, producers, ring
#ifndef SPTRSV_GRID_CHK
#define SPTRSV_GRID_CHK 4
#endif
// consumer steps per ring check (a divisor of kGridBlk, even): half blocks for 2D stencils (c3 0.795 ->
// 0.776 ms, 2 steps: 0.803), whole blocks with far entries (3D: 4.49 vs 4.62 ms at 4)
constexpr int kGridChk2D = SPTRSV_GRID_CHK;
static_assert(kGridBlk % kGridChk2D == 0 && kGridChk2D % 2 == 0, "ring checks tile the block in step pairs");
#ifndef SPTRSV_GRID_RING_WARP
#define SPTRSV_GRID_RING_WARP 4
#endif
constexpr int kGridRingWarp = SPTRSV_GRID_RING_WARP;  // (kGridWarps - 1 puts it on its own)
static_assert(kGridA1 == 2 * kGridA2, "one cp.async wait covers both staging distances");
static_assert(kGridBlk * (kGridA1 + 1) <= kGridRaw, "raw ring too small");

enum : int { kDescN = 2, kDescW = 4, kDescFar = 8 /* far entry not folded: poll it */ };

__host__ __device__ constexpr size_t grid_smem_bytes(int ecap) {
    return (size_t)kGridDesc * 32 * 64 + (size_t)kGridDesc * 8 +
           (size_t)kGridRaw * (64 * 4 + 32 * 8 + (size_t)ecap * 12);
}

__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void cp_async4(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async8(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }


// the rare in-loop division outside the guard (zero numerators, extreme magnitudes): out of line, so the
// step's hot path carries no divergent branch
__device__ __noinline__ double grid_fix_div(bool fix, double a, double d, double q) {
    return fix ? __ddiv_rn(a, d) : q;
}

// the consumer / producer barrier (named barrier 1, warps 0 .. kGridProd; the ring warp runs free)
__device__ __forceinline__ void bar_sync_cp() {
    asm volatile("bar.sync 1, %0;" ::"n"(32 * (1 + kGridProd)) : "memory");
}
__device__ __forceinline__ int ld_volatile_s32(const int *a) {
    int v;
    asm volatile("ld.volatile.shared.s32 %0, [%1];" : "=r"(v) : "r"((unsigned)__cvta_generic_to_shared(a)) : "memory");
    return v;
}
__device__ __forceinline__ void st_volatile_s32(int *a, int v) {
    asm volatile("st.volatile.shared.s32 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(a)), "r"(v) : "memory");
}

// GRID's publishes: predicated stores WITHOUT a compiler memory clobber, so the scheduler may overlap
// them with the next step's shared-memory loads (they only depend on the quotient)
__device__ __forceinline__ void grid_st_rec_if(bool pr, unsigned long long *a, unsigned long long lo,
                                               unsigned long long hi) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\t@q st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};\n\t}" ::"l"(a),
                 "l"(lo), "l"(hi), "r"((unsigned)pr));
}
__device__ __forceinline__ void grid_st_x_if(bool pr, unsigned long long *a, unsigned long long v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q st.global.u64 [%0], %1;\n\t}" ::"l"(a), "l"(v),
                 "r"((unsigned)pr));
}
__device__ __forceinline__ int ld_volatile_s32_nc(const int *a) {  // no compiler memory clobber
    int v;
    asm volatile("ld.volatile.shared.s32 %0, [%1];" : "=r"(v) : "r"((unsigned)__cvta_generic_to_shared(a)));
    return v;
}

// FAR: the matrix has far entries (7-point-like stencils); without them the step carries no far-entry
// code at all (one basic block less per step for the scheduler)
// UPPER / UNIT: the triangular forms (GridForm above): bands, lines and columns are logical; the CSR
// slice of a band's logical line is a contiguous run of physical rows (reversed for upper handles,
// which analyse admits only when n is a multiple of m); b, x and the records are physical.
template <int PROTO, bool SAFE, bool FAR, bool UPPER = false, bool UNIT = false>
__global__ void __launch_bounds__(32 * kGridWarps, 1) k_solve_grid(SolveParams p) {
    extern __shared__ __align__(16) unsigned char gsm[];
    __shared__ uint32_t s_blk, s_epoch, s_stop;
    __shared__ int s_ring, s_cons;  // lines whose west value is in s_west; the consumer's block start
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        cta_ticket(p, s_blk, s_epoch);
        s_stop = 0;
        s_ring = 0;
        s_cons = 0;
    }
    __syncthreads();
    if (s_blk == kStaleBlk) return;
    const uint32_t epoch = s_epoch;
    const int m = p.grid_m, lines = p.grid_lines, E = p.grid_ecap;
    const unsigned n = (unsigned)p.n;
    const int band = (int)s_blk;
    const int x0 = band * 32;
    const int nl = min(32, m - x0);  // lanes owning a column (>= 1: the grid is ceil(m / 32) bands)
    const int steps = lines + nl - 1;
    const int nblocks = (steps + kGridBlk - 1) / kGridBlk;
    // ---- shared memory: descriptor ring, then raw ring
    // descriptors, [desc][32] 16-byte pairs (one 128-bit shared load each): {ls0 (far product summed, or
    // vf if pending), vn}, {vw, b}, {d, RN(1/d)}, {meta, far column, row (-1 = none), 0}
    double2 *d_a = reinterpret_cast<double2 *>(gsm);
    double2 *d_bw = d_a + kGridDesc * 32, *d_dr = d_bw + kGridDesc * 32;
    int4 *d_m = reinterpret_cast<int4 *>(d_dr + kGridDesc * 32);
    double *s_west = reinterpret_cast<double *>(d_m + kGridDesc * 32);     // [desc]: lane 0's west x
    int32_t *s_rp = reinterpret_cast<int32_t *>(s_west + kGridDesc);        // [raw][64]
    double *s_b = reinterpret_cast<double *>(s_rp + kGridRaw * 64);          // [raw][32]
    double *s_val = s_b + kGridRaw * 32;                                     // [raw][E]
    int32_t *s_col = reinterpret_cast<int32_t *>(s_val + (size_t)kGridRaw * E);  // [raw][E]

    const bool ring_on = band > 0;
    // warp roles: 0 consumer, kGridRingWarp the ring, the others producers (SM sub-partition = warp % 4:
    // the ring warp, mostly waiting on its polls, shares the consumer's sub-partition)
    if (warp == kGridRingWarp) {
        // ================================================================ the ring (band > 0)
        // Lane 0's west operand is band k-1's lane 31: this warp polls those records 32 lines at a
        // time (lane j: line base + j), stores the values of the ready prefix in s_west and advances
        // s_ring, one round trip per pass -- the consumer only reads shared memory.  It stays within
        // kGridDesc - 8 lines of the consumer's block start (s_west's slots).
        if (!ring_on) return;
        int base = 0;
        uint32_t bo = p.backoff_min, idl = 0;
        while (base < lines) {
            const int y = base + lane;
            const unsigned wl = (unsigned)y * (unsigned)m + (unsigned)x0 - 1u;  // logical west row
            const bool need = y < lines && wl < n;
            const unsigned wr = UPPER ? n - 1u - wl : wl;                       // its physical row
            const bool room = y < ld_volatile_s32(&s_cons) + kGridDesc - 8;
            unsigned long long w0 = 0, w1 = 0;
            if (need && room) poll1<PROTO>(p, (int)wr, w0, w1);
            const bool rdy = room && (!need || ready1<PROTO>(w0, w1, epoch));
            const unsigned mask = __ballot_sync(FULL, rdy);
            const int L = __ffs(~mask) - 1 < 0 ? 32 : __ffs(~mask) - 1;  // ready prefix
            if (lane < L && need) s_west[y % kGridDesc] = value1<PROTO>(p, (int)wr, w0, w1);
#ifdef SPTRSV_GRID_TRACE  // measurement builds only: when the ring warp stored line y's west value
            if (p.trace && lane < L && need) p.trace[(size_t)n + (size_t)y * ((m + 31) / 32) + band] = globaltimer_ns();
#endif
            __syncwarp();
            if (L > 0) {
                __threadfence_block();
                if (lane == 0) st_volatile_s32(&s_ring, base + L);
                base += L;
                bo = p.backoff_min;
                idl = 0;
                continue;
            }
            if (ld_volatile_s32((const int *)&s_stop)) return;
            if (bo) nanosleep_ns(bo);
            bo = min(max(bo * 2u, 32u), p.backoff_max);
            ++idl;
            if ((idl & 63u) == 0 || (p.spin_limit && idl >= p.spin_limit)) {
                uint32_t ab = 0;
                if (lane == 0) {
                    if (p.spin_limit && idl >= p.spin_limit) {
                        atomicCAS(&p.st->error.v, 0u, kErrTimeout);
                        st_relaxed_u32(&p.st->abort.v, 1u);
                    }
                    ab = ld_relaxed_u32(&p.st->abort.v);
                }
                if (__shfl_sync(FULL, ab, 0)) {
                    if (lane == 0) st_volatile_s32((int *)&s_stop, 1);
                    return;
                }
            }
        }
        return;
    }
    if (warp > 0) {
        // ================================================================ producers
        const int w = warp < kGridRingWarp ? warp - 1 : warp - 2;
        // rows of logical line y in this band (0: none); row0 = the first PHYSICAL row of its CSR slice
        // (upper: logical row y*m + x0 + j is physical n-1-(y*m + x0 + j), so the slice runs backwards)
        auto line_rows = [&](int y, unsigned &row0) -> int {
            const unsigned l0 = (unsigned)y * (unsigned)m + (unsigned)x0;
            if (y < 0 || y >= lines || l0 >= n) return 0;
            const int k = min(nl, (int)(n - l0));
            row0 = UPPER ? n - l0 - (unsigned)k : l0;
            return k;
        };
        auto stage_rp = [&](int y) {  // rowptr[row0 .. row0 + k] and b[row0 .. row0 + k)
            unsigned row0;
            const int k = line_rows(y, row0);
            if (k == 0) return;
            int32_t *rp = s_rp + (y & (kGridRaw - 1)) * 64;
            if (lane <= k) cp_async4(rp + lane, p.rowptr + row0 + lane);
            if (lane == 0 && k == 32) cp_async4(rp + 32, p.rowptr + row0 + 32);
            if (lane < k) cp_async8(s_b + (y & (kGridRaw - 1)) * 32 + lane, p.b + row0 + lane);
        };
        auto stage_ent = [&](int y) {  // entries of line y (its rowptr slice complete in the ring)
            unsigned row0;
            const int k = line_rows(y, row0);
            if (k == 0) return;
            const int sl = y & (kGridRaw - 1);
            const int lo = s_rp[sl * 64], hi = s_rp[sl * 64 + k];
            for (int e = lo + lane; e < hi; e += 32) {
                cp_async4(s_col + (size_t)sl * E + (e - lo), p.colidx + e);
                cp_async8(s_val + (size_t)sl * E + (e - lo), p.val + e);
            }
        };
        // descriptors of line y from its staged raw rows; lines outside [0, lines) (the skew's head and
        // tail: line s - lane) get inactive descriptors (row -1, no entries), so the consumer reads them
        // without a range check
        auto produce = [&](int y) {
            unsigned row0 = 0;
            const int k = line_rows(y, row0);
            const int sl = y & (kGridRaw - 1), ds = ((y + kGridDesc) % kGridDesc) * 32 + lane;
            const bool act = lane < k;
            const int pj = UPPER ? k - 1 - lane : lane;  // this lane's row in the (physical) slice
            const int r = (int)(row0 + pj);              // physical row
            const int rl = (int)((unsigned)y * (unsigned)m + (unsigned)x0) + lane;  // logical row
            const GridForm gf{UPPER, UNIT, (int32_t)n};
            int meta = 0, fc = 0;
            double ls0 = 0.0, vn = 0.0, vw = 0.0, bv = 0.0, dv = 1.0, rc = 1.0;
            if (act) {
                const int base = s_rp[sl * 64];
                int lo, hi;
                gf.offdiag(s_rp[sl * 64 + pj] - base, s_rp[sl * 64 + pj + 1] - base, lo, hi);
                const double *v = s_val + (size_t)sl * E;
                const int32_t *c = s_col + (size_t)sl * E;
                const int cnt = hi - lo;
                // off-diagonals counted from the logically last one: west (rl - 1), north (rl - m), far
                const int jw = gf.from_last(lo, hi, 0);
                const bool hw = cnt > 0 && gf.logical(c[jw]) == rl - 1;  // (row 0 has no west)
                const int jn = gf.from_last(lo, hi, (int)hw);
                const bool hn = cnt > (int)hw && gf.logical(c[jn]) == rl - m;
                const int tf = (int)hw + (int)hn;
                const int jf = gf.from_last(lo, hi, tf);
                meta = (hn ? kDescN : 0) | (hw ? kDescW : 0);
                vw = hw ? v[jw] : 0.0;
                vn = hn ? v[jn] : 0.0;
                if (FAR && cnt > tf) {  // the far entry (at most one: k_grid_check)
                    fc = c[jf];  // physical: the records are indexed by physical row
                    const double vf = v[jf];
                    unsigned long long f0, f1;
                    poll1<PROTO>(p, fc, f0, f1);
                    if (ready1<PROTO>(f0, f1, epoch)) {
                        ls0 = __dadd_rn(0.0, __dmul_rn(vf, value1<PROTO>(p, fc, f0, f1)));
                    } else {
                        ls0 = vf;
                        meta |= kDescFar;
                    }
                }
                bv = s_b[sl * 32 + pj];
                Diag g;
                g.init(UNIT ? 1.0 : v[UPPER ? s_rp[sl * 64 + pj] - base : s_rp[sl * 64 + pj + 1] - base - 1]);
                dv = g.d;
                rc = g.r;
            }
            d_a[ds] = make_double2(ls0, vn);
            d_bw[ds] = make_double2(vw, bv);
            d_dr[ds] = make_double2(dv, rc);
            d_m[ds] = make_int4(meta, fc, act ? r : -1, 0);
        };
        // prologue: the raw rows of the first lines, then the descriptors of lines [0, kGridBlk]
        for (int y = w; y < kGridBlk + 1 + kGridBlk * kGridA1; y += kGridProd) stage_rp(y);
        cp_async_commit();
        cp_async_wait<0>();
        __syncwarp();
        for (int y = w; y < kGridBlk + 1 + kGridBlk * kGridA2; y += kGridProd) stage_ent(y);
        cp_async_commit();
        cp_async_wait<0>();
        __syncwarp();
        // lines -31 .. -1 (the head: inactive) and 0 .. kGridBlk; a line >= 0 is produced by the warp that
        // staged it (y = w mod kGridProd: cp.async completion is per thread, no CTA barrier yet)
        static_assert(32 % kGridProd == 0, "the head loop keeps each warp's staged lines");
        for (int y = w - 32; y <= kGridBlk; y += kGridProd)
            if (y > -32) produce(y);
        for (int b = 0; b < nblocks; ++b) {
            bar_sync_cp();  // block b begins: lines <= B*b + B are in the descriptor ring
            if (ld_volatile_s32((const int *)&s_stop)) continue;
            cp_async_wait<kGridA2 - 1>();
            __syncwarp();
            const int y0 = kGridBlk * b + kGridBlk + 1;
            static_assert(kGridBlk % kGridProd == 0, "each producer: the same number of lines per block");
#pragma unroll
            for (int i = 0; i < kGridBlk / kGridProd; ++i) {
                stage_rp(y0 + w + i * kGridProd + kGridBlk * kGridA1);
                stage_ent(y0 + w + i * kGridProd + kGridBlk * kGridA2);
            }
            cp_async_commit();
#pragma unroll
            for (int i = 0; i < kGridBlk / kGridProd; ++i) produce(y0 + w + i * kGridProd);
        }
        cp_async_wait<0>();
        return;
    }
    // ==================================================================== consumer (warp 0)
    // the row of a step (line s - lane) comes from the descriptor ring through a per-lane cursor (the
    // byte offset of its ring slot's d_a pair), advanced once per step; the NEXT step's row is fetched at
    // the top of each step so its shared-memory loads overlap the current chain
    constexpr unsigned kSlotB = 32 * sizeof(double2), kArrB = kGridDesc * kSlotB;
    const unsigned fwrap = kArrB + 16u * lane;  // one past the last slot
    unsigned fad = (lane == 0 ? 0u : (unsigned)(kGridDesc - lane) * kSlotB) + 16u * lane;
    struct Row {
        int r, meta, fc;
        double ls0, vn, vw, b, d, rc;
    };
    auto fetch = [&](Row &o) {
        const unsigned char *sp = gsm + fad;  // d_a, d_bw, d_dr, d_m: consecutive [desc][32] arrays
        const int4 mm = *reinterpret_cast<const int4 *>(sp + 3 * kArrB);
        const double2 a2 = *reinterpret_cast<const double2 *>(sp);
        const double2 bw = *reinterpret_cast<const double2 *>(sp + kArrB);
        const double2 dr = *reinterpret_cast<const double2 *>(sp + 2 * kArrB);
        o.r = mm.z;
        o.meta = mm.x;
        o.ls0 = a2.x;
        o.vn = a2.y;
        o.vw = bw.x;
        o.b = bw.y;
        o.d = dr.x;
        o.rc = dr.y;
        o.fc = mm.y;
        fad += kSlotB;
        fad = fad == fwrap ? 16u * lane : fad;
    };
    double xl = 0.0;   // this lane's latest x (the north operand of its next row)
    double xsh = 0.0;  // the west lane's latest x, shuffled as soon as it was computed (next step's west)
    bool bad = false, stop = false;
    int ring_have = ring_on ? 0 : 0x7fffffff;  // lines whose west value the ring warp has stored
    const unsigned long long ep = (unsigned long long)epoch << 32;
    // the rare cases wait here: the ring behind (lane 0's west not stored yet), or a far entry that was
    // not published when its row was produced (polled in place); backoff and watchdog as everywhere
    auto wait_for = [&](int s, bool pend, int fc, double &xf) -> bool {
        uint32_t bo = p.backoff_min, idl = 0;
        bool have_f = !pend;
        while (true) {
            if (ring_have <= s) ring_have = ld_volatile_s32(&s_ring);
            if (!have_f) {
                unsigned long long f0, f1;
                poll1<PROTO>(p, fc, f0, f1);
                if (ready1<PROTO>(f0, f1, epoch)) {
                    xf = value1<PROTO>(p, fc, f0, f1);
                    have_f = true;
                }
            }
            if (!__any_sync(FULL, ring_have <= s || !have_f)) return true;
            if (ld_volatile_s32((const int *)&s_stop)) return false;
            if (bo) nanosleep_ns(bo);
            bo = min(max(bo * 2u, 32u), p.backoff_max);
            ++idl;
            if ((idl & 63u) == 0 || (p.spin_limit && idl >= p.spin_limit)) {
                uint32_t ab = 0;
                if (lane == 0) {
                    if (p.spin_limit && idl >= p.spin_limit) {
                        atomicCAS(&p.st->error.v, 0u, kErrTimeout);
                        st_relaxed_u32(&p.st->abort.v, 1u);
                    }
                    ab = ld_relaxed_u32(&p.st->abort.v);
                }
                if (__shfl_sync(FULL, ab, 0)) return false;
            }
        }
    };
    constexpr bool has_far = FAR;
    // one step (line s - lane; lane 0's west value wv): Alg.1's row, the division, the publish.  `cur` is
    // this step's row, `nxt` receives the next one (two register sets alternate)
    auto step = [&](Row &cur, Row &nxt, int s, double wv) -> bool {
        fetch(nxt);  // the next step's row (its lines were produced before this block)
        const int r = cur.r;
        const bool act = r >= 0;
        const bool pend = has_far && (cur.meta & kDescFar) != 0;
        double xf = 0.0;
        if (has_far && __any_sync(FULL, pend)) {  // a far entry not published when its row was produced
            if (!wait_for(-1, pend, cur.fc, xf)) return false;
        }
        const double xw = lane == 0 ? wv : xsh;
        // ---- Alg.1's row: far (ls0), north, west (column order), then the division
        double ls = pend ? __dadd_rn(0.0, __dmul_rn(cur.ls0, xf)) : cur.ls0;
        ls = (cur.meta & kDescN) ? __dadd_rn(ls, __dmul_rn(cur.vn, xl)) : ls;
        ls = (cur.meta & kDescW) ? __dadd_rn(ls, __dmul_rn(cur.vw, xw)) : ls;
        const double a = __dsub_rn(cur.b, ls);
        Diag g;
        g.d = cur.d;
        g.r = cur.rc;
        double q = g.cand(a);
        const bool guard = Diag::in_range(a) && cur.rc != 0.0;
        if (SAFE) {
            const bool fix = act && !(guard && Diag::exact(a, cur.d, q));
            if (__builtin_expect(__any_sync(FULL, fix), 0)) q = grid_fix_div(fix, a, cur.d, q);
            xsh = __shfl_up_sync(FULL, q, 1);
        } else {
            // outside the guard (a zero numerator, extreme magnitudes): the full division, in-loop;
            // inside it the candidate's proof runs off the chain and a failure fails the solve
            const bool fix = act && !guard;
            if (__builtin_expect(__any_sync(FULL, fix), 0)) q = grid_fix_div(fix, a, cur.d, q);
            xsh = __shfl_up_sync(FULL, q, 1);  // first: the next step's chain starts here
            // (bitwise: the proof runs unconditionally, no branch around it in the step)
            const bool ex = Diag::exact(a, cur.d, q);
            bad = bad | (act & guard & !ex);
        }
        // ---- publish (Alg.5 l.13-16); GRID records are read by GRID warps only (no shared-memory
        // sentinel to avoid)
        const int ri = r;  // (an inactive row's -1 only forms the address of a predicated-off store)
#ifdef SPTRSV_GRID_M_NOSTORE  // measurement builds only (tools/)
        if (false) {
#else
        if (PROTO == PROTO_FUSED) {
#endif
            const unsigned long long bits = (unsigned long long)__double_as_longlong(q);
            grid_st_rec_if(act, p.rec + 2 * (size_t)ri, ep | (bits & 0xffffffffull), ep | (bits >> 32));
            grid_st_x_if(act, reinterpret_cast<unsigned long long *>(p.x) + ri, bits);
        } else if (act) {
            p.x[r] = q;
            st_release_u32(p.flags + r, epoch);
        }
        // unconditionally: a lane's x is read (as its next row's north, or its east neighbour's west)
        // only by active rows, and an active row's predecessor step on this lane / the west lane is active
        // too (lines start and end on the skew: line s - l; rows past n, lanes past nl stay inactive)
        xl = q;
#ifdef SPTRSV_GRID_TRACE  // measurement builds only (tools/grid_trace.py): publish time of every row
        if (p.trace && act) p.trace[r] = globaltimer_ns();
#endif
        return true;
    };
    Row ra, rb;
    int wbase = 0;  // (kGridBlk * b) mod kGridDesc: s_west slot of the block's first step
    static_assert(kGridDesc % kGridBlk == 0 && kGridBlk % 2 == 0, "block steps tile the west ring");
    for (int b = 0; b < nblocks; ++b) {
        if (lane == 0) st_volatile_s32(&s_cons, kGridBlk * b);
        bar_sync_cp();
        if (stop) continue;
        if (b == 0) fetch(ra);
        const int s0 = kGridBlk * b;
        const int s_end = min(steps, s0 + kGridBlk);
        // lane 0's west values, kGridChk steps at a time (the ring warp stores lines in chunks), waiting
        // only when the ring is behind; a check inside the block runs after the previous step's shuffle
        auto ring_check = [&](int need) -> bool {
            if (ring_have <= need) ring_have = ld_volatile_s32_nc(&s_ring);
            if (ring_have <= need) {
                double dummy;
                if (!wait_for(need, false, 0, dummy)) return false;
            }
            asm volatile("" ::: "memory");  // the s_west loads stay after the s_ring check
            return true;
        };
        constexpr int kGridChk = FAR ? kGridBlk : kGridChk2D;
        const bool full = s_end - s0 == kGridBlk;
        if (!ring_check(min(full ? s0 + kGridChk : s_end, lines) - 1)) stop = true;
        if (!stop) {
            if (full) {
                double wblk[kGridBlk];
#pragma unroll
                for (int k = 0; k < kGridBlk; k += 2) {
                    if (k % kGridChk == 0) {
                        if (k > 0 && !ring_check(min(s0 + k + kGridChk, lines) - 1)) {
                            stop = true;
                            break;
                        }
                        // lane 0's west values of the next kGridChk steps (16-byte aligned pairs)
#pragma unroll
                        for (int j = k; j < k + kGridChk; j += 2) {
                            const double2 w2 = *reinterpret_cast<const double2 *>(s_west + wbase + j);
                            wblk[j] = w2.x;
                            wblk[j + 1] = w2.y;
                        }
                    }
                    if (!step(ra, rb, s0 + k, wblk[k]) || !step(rb, ra, s0 + k + 1, wblk[k + 1])) {
                        stop = true;
                        break;
                    }
                }
            } else {  // the last, partial block
                for (int k = 0; k < s_end - s0; ++k) {
                    Row &c = (k & 1) ? rb : ra;
                    Row &nx = (k & 1) ? ra : rb;
                    if (!step(c, nx, s0 + k, s_west[wbase + k])) {
                        stop = true;
                        break;
                    }
                }
            }
        }
        wbase = wbase + kGridBlk == kGridDesc ? 0 : wbase + kGridBlk;
        if (stop && lane == 0) st_volatile_s32((int *)&s_stop, 1);  // producers and ring skip the rest
    }
    if (lane == 0) st_volatile_s32(&s_cons, 0x3fffffff);
    if (!stop && !SAFE && __any_sync(FULL, bad || p.chain_div == 2)) {
        if (lane == 0) {
            atomicCAS(&p.st->error.v, 0u, kErrInexact);
            st_relaxed_u32(&p.st->abort.v, 1u);
        }
    }
}

}  // namespace sptrsv_dev
