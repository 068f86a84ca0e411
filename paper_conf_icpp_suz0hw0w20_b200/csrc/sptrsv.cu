// sptrsv.cu -- host side of the C ABI declared in include/sptrsv.h.
//
// Torch-free: raw device pointers and cudaStream_t only.  Built as
// libsptrsv.so for sm_100a (see paper_conf_icpp_suz0hw0w20_b200/build.py).
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>

#include "diag.cuh"
#include "setup.cuh"
#include "solve.cuh"
#include "solve_lean.cuh"
#include "solve_tri.cuh"
#include "solve_multi.cuh"
#include "solve_paper.cuh"
#include "solve_chain.cuh"
#include "solve_small.cuh"
#include "solve_grid.cuh"
#include "sptrsv.h"

using namespace sptrsv_dev;

namespace {

constexpr uint32_t kEpochResetAt = 0xFFFFFF00u;  // re-zero the flags before the epoch wraps

// engines (SPTRSV_OPT_ENGINE values, include/sptrsv.h)
enum { ENG_ONESHOT = 0, ENG_LEAN = 3, ENG_AUTO = 5, ENG_HYBRID = 6, ENG_CHAIN = 7, ENG_SMALL = 8, ENG_LEANP = 9, ENG_GRID = 10 };

// ENGINE_SMALL (solve_small.cuh): the whole system in one CTA's shared memory.  Usable when it fits
// (kSmallSmemMax bytes of dynamic shared memory, sm_100a allows 227 KB per CTA); AUTO picks it up to
// kSmallAutoN rows (measured against LEAN / ONE-SHOT / CHAIN on c1-shaped systems).
constexpr size_t kSmallSmemMax = 226 * 1024;
constexpr int kSmallAutoN = 4096;
constexpr int kSmallCta = 256;

// The handle's workspace is ONE device allocation (analyse is O(nnz) work plus a fixed handful of
// runtime calls), carved in 256-byte aligned pieces: the 16-byte FUSED records, the FLAGS words,
// in-degrees, the task list (at most n tasks), the solve state and the analyse results / scratch.
struct Workspace {
    void *base = nullptr;          // the single allocation below
    bool pooled = false;           // from the library's memory pool (ws_pool) rather than cudaMalloc
    uint32_t *flags = nullptr;     // n      (PROTO_FLAGS)
    unsigned long long *rec = nullptr;  // 2n (PROTO_FUSED)
    int32_t *indeg = nullptr;      // n
    int32_t *tasks = nullptr;      // n (PLAN_LIST uses n_tasks <= n of them)
    uint8_t *task_w = nullptr;     // n: lanes per row of each task (0 thread group, 32 warp row, 2..16)
    SolveState *st = nullptr;      // 1
    AnalyseOut *aout = nullptr;    // 1: analyse results (one D2H copy)
    int32_t *blk = nullptr;        // 3 * nb: plan block counts / thread groups / offsets
    uint32_t *lvl = nullptr;       // n (levels diagnostic, lazy)
    double *b_stage = nullptr;     // n (solve_host, lazy)
    SolveState *mst = nullptr;     // multi-RHS: own solve state (own epoch sequence)
    // sptrsv_solve_host on a LEANP handle runs the LEAN kernel (its per-CTA b gating and x write-back
    // overlap the PCIe copies better: c2 e2e 270 vs 305 us) on its OWN ready words and epoch sequence,
    // so host and device solves interleave without re-zeroing each other's state (lazy)
    SolveState *hst = nullptr;
    unsigned long long *hrec = nullptr;  // 2n
    uint32_t *hflags = nullptr;          // n
    uint32_t *mflags = nullptr;    // multi-RHS: n * mcap flags (FLAGS)
    unsigned long long *mrec = nullptr;  // multi-RHS: n * mcap records (FUSED)
    int64_t mcap = 0;              // right-hand sides the multi buffers hold
    double *x_stage = nullptr;     // n (solve_host, lazy)
    uint32_t *bflag = nullptr;     // solve_host: per-chunk "b has landed" words (lazy)
    int32_t bflag_n = 0;
    cudaStream_t s2 = nullptr;     // solve_host: copy stream for the chunked b
    cudaEvent_t ev_a = nullptr, ev_b = nullptr;
    cudaEvent_t ev_done = nullptr;  // solve_host: completion (spin_sync)
};

// cuStreamWriteValue32 through the runtime's driver entry point (no link-time libcuda
// dependency: the library must load on machines without a GPU driver).
typedef int (*write_value32_fn)(cudaStream_t, unsigned long long, uint32_t, unsigned int);
write_value32_fn write_value32() {
    static write_value32_fn fn = [] {
        void *f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &f, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess) {
            (void)cudaGetLastError();
            f = nullptr;
        }
        return (write_value32_fn)f;
    }();
    return fn;
}
constexpr int kBChunkShift = 16;  // solve_host: smallest b chunk, 2^16 rows (512 KB)

// sptrsv_solve_host's completion wait: an event on the stream polled by the calling thread (a
// blocking cudaStreamSynchronize may yield the thread and add its wake-up to every end-to-end step)
int spin_sync(cudaStream_t s, cudaEvent_t &ev) {
    if (!ev && cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess) {
        (void)cudaGetLastError();
        return cudaStreamSynchronize(s) == cudaSuccess ? 0 : -1;
    }
    if (cudaEventRecord(ev, s) != cudaSuccess) return -1;
    cudaError_t e;
    while ((e = cudaEventQuery(ev)) == cudaErrorNotReady) {
    }
    return e == cudaSuccess ? 0 : -1;
}

}  // namespace

struct sptrsv_handle_s {
    int device = 0;
    // sptrsv_analyse_csr_batch: the handle owns the block-diagonal concatenation of its systems
    int32_t *own_rowptr = nullptr, *own_colidx = nullptr;
    double *own_val = nullptr;
    int32_t n = 0;
    int64_t nnz = 0;
    const int32_t *rowptr = nullptr;
    const int32_t *colidx = nullptr;
    const double *val = nullptr;
    Workspace ws;
    // plan
    int plan = PLAN_THREAD;
    int32_t n_tasks = 0;
    int32_t n_tasks_cap = 0;
    int32_t n_thread_groups = 0;
    int32_t n_warp_rows = 0;
    int32_t n_sub_tasks = 0;  // tasks of 2..16 lanes per row (sub-warp rows)
    int subwarp_epl = -1;     // SPTRSV_OPT_SUBWARP: off-diagonals per lane of a sub-warp row (-1 AUTO, 0 off)
    int epl_eff = 0;          // the value the current plan used
    int32_t max_row = 0;
    int64_t near_deps = 0;  // dependencies within 256 rows (analyse statistic for ENGINE_AUTO)
    int64_t warp_deps = 0;  // dependencies inside the row's own 32-row group (ditto)
    int64_t prev_deps = 0;  // dependencies on the previous row in solve order (ditto: chains)
    int64_t mid_breaks = 0; // rows off a 64-row boundary without a previous-row dependency (ditto)
    int64_t near_rows = 0;  // rows whose nearest dependency is < 256 rows away (ditto)
    int32_t grid_m = 0;     // ENGINE_GRID: line length found by analyse (0 = none), rows violating its
    int32_t grid_viol = 0;  // band order, north / west entries and far entries (solve_grid.cuh)
    int64_t grid_fast = 0, grid_far = 0;
    // options
    int mode = 0;
    int threshold = 16;
    bool threshold_user = false;  // SPTRSV_OPT_WARP_THRESHOLD set explicitly
    int dmin_log2 = -1;           // floor(log2(median nearest-dependency distance)), -1 = no dependencies
    int cta_threads = 0;    // 0 = per-engine default (see plan_launch)
    uint32_t backoff_min = 0;
    uint32_t backoff_max = 256;
    uint32_t spin_limit = 1u << 24;
    int l2_window = 1;      // persisting L2 window over the ready words (SPTRSV_OPT_L2_WINDOW)
    float l2_hit = 0.f;     // its hitRatio once the set-aside is sized (0 = not yet)
    bool l2_user = false;   // counted among the device's persisting-L2 users (l2_limit_*)
    int stage = 1;
    int proto = PROTO_FUSED;
    int local = 1;
    int engine = ENG_AUTO;  // SPTRSV_OPT_ENGINE: ENG_AUTO or a forced engine (resolve_engine)
    int rows_per_lane = 0;  // CHAIN: K rows per lane (0 = 2)
    int variant = 0;        // 0 product path; 3 / 4 / 5 = the paper's Alg.3 / Alg.4 / Alg.5 (ablation)
    int lean_minb = 5;      // LEAN: resident 256-thread CTAs per SM the register budget targets (5..8)
    uint32_t poll_gap = 0;  // LEAN: sleep after a progressing pass (SPTRSV_OPT_POLL_GAP_NS)
    int poll_one = 0;       // LEAN: one poll per lane per pass (SPTRSV_OPT_POLL_ONE)
    int host_io = 3;        // sptrsv_solve_host on LEAN with pinned buffers (SPTRSV_OPT_HOST_IO)
    uint32_t host_seq = 0;  // solve_host: sequence number of the chunked-b flags
    int split_last = 2;     // warp rows: last off-diagonal outside the lane tree (SPTRSV_OPT_WARP_SPLIT_LAST)
    int chain_div = 0;      // SPTRSV_OPT_CHAIN_DIV: 0 proof after each run, 1 in-loop proof, 2 test hook
    int tri = 0;            // SPTRSV_TRI_* flags of sptrsv_analyse_csr_ex (f4): 1 UPPER, 2 UNIT_DIAG
    int grid_cache_key = -1;
    int grid_cache = 0;
    int launch_key = -1;  // configuration of the last launch (see sptrsv_solve)
    long long mlaunch_key = -1;  // same for sptrsv_solve_multi
    uint32_t msince_reset = 0;
    uint32_t gen = 0, mgen = 0;  // configuration generations of the solve / multi-RHS state (cta_ticket)
    uint32_t hgen = 0, hsince_reset = 0;  // the host-path state (Workspace::hst)
    int hlaunch_key = -1;
    bool no_coop = false;  // a cooperative launch was refused (shared GPU, MPS): AUTO falls back to LEAN
    unsigned long long *trace = nullptr;
    // bookkeeping
    uint32_t solves = 0;
    uint32_t since_reset = 0;
    float analyse_ms = 0.f;
};

namespace {
// The persisting-L2 set-aside is a device-wide limit.  The library grows it for handles whose
// ready-word window it can hold, remembers the value it found, and restores that value when the
// last handle using a window on the device is destroyed (or turns its window off), so a host
// application's L2 is only shared while a windowed handle exists.
struct L2Limit {
    size_t orig = 0;
    int users = 0;
};
std::mutex g_l2_mu;
L2Limit g_l2[256];

void l2_limit_release(sptrsv_handle_s *h);
}  // namespace

// Makes a handle's device current for a host entry point and restores the caller's on exit.
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) cudaSetDevice(dev);
        (void)cudaGetLastError();
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
        (void)cudaGetLastError();
    }
};

#define CK(call)                                        \
    do {                                                \
        if ((call) != cudaSuccess) {                    \
            (void)cudaGetLastError();                   \
            return SPTRSV_ERR_CUDA;                     \
        }                                               \
    } while (0)

namespace {

void l2_limit_release(sptrsv_handle_s *h) {
    std::lock_guard<std::mutex> lk(g_l2_mu);
    if (!h->l2_user) return;
    h->l2_user = false;
    L2Limit &e = g_l2[h->device & 255];
    if (--e.users == 0) {
        (void)cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, e.orig);
        (void)cudaGetLastError();
        e.orig = 0;
    }
}

// dynamic smem: x copy [warps*32] doubles, then (if staging) [warps][kStageCap] doubles + ints
size_t solve_smem_bytes(int cta_threads, int stage) {
    const size_t w = (size_t)(cta_threads / 32);
    return w * 32 * sizeof(double) + (stage ? w * kStageCap * (sizeof(double) + sizeof(int32_t)) : 0);
}

typedef void (*solve_fn)(SolveParams);
solve_fn solve_kernel(int plan, int proto) {
    static const solve_fn tab[3][2] = {
        {k_solve<PLAN_THREAD, PROTO_FLAGS>, k_solve<PLAN_THREAD, PROTO_FUSED>},
        {k_solve<PLAN_WARP, PROTO_FLAGS>, k_solve<PLAN_WARP, PROTO_FUSED>},
        {k_solve<PLAN_LIST, PROTO_FLAGS>, k_solve<PLAN_LIST, PROTO_FUSED>},
    };
    return tab[plan][proto];
}

int set_kernel_attrs() {
    static int done = 0;
    static int rc = SPTRSV_OK;
    if (done) return rc;
    const int maxb = (int)solve_smem_bytes(1024, 1);
    for (int pl = 0; pl < 3; ++pl)
        for (int pr = 0; pr < 2; ++pr)
            if (cudaFuncSetAttribute(solve_kernel(pl, pr), cudaFuncAttributeMaxDynamicSharedMemorySize, maxb) !=
                cudaSuccess) {
                (void)cudaGetLastError();
                rc = SPTRSV_ERR_CUDA;
            }
    done = 1;
    return rc;
}

// Handle workspaces come from a library-private stream-ordered memory pool per device: a destroyed
// handle's workspace is kept (up to kPoolKeepBytes) and handed to the next analyse without a
// cudaMalloc / cudaFree pair -- the warm analyse is then a memset, six kernels and one copy.
constexpr unsigned long long kPoolKeepBytes = 1ull << 30;
std::mutex g_pool_mu;
cudaMemPool_t g_pool[256] = {};

cudaMemPool_t ws_pool(int dev) {
    std::lock_guard<std::mutex> lk(g_pool_mu);
    cudaMemPool_t &p = g_pool[dev & 255];
    if (!p) {
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        if (cudaMemPoolCreate(&p, &props) != cudaSuccess) {
            (void)cudaGetLastError();
            p = nullptr;
            return nullptr;
        }
        unsigned long long keep = kPoolKeepBytes;
        (void)cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &keep);
        (void)cudaGetLastError();
    }
    return p;
}

void free_ws(Workspace &w) {
    if (w.base) {
        if (w.pooled) {
            (void)cudaFreeAsync(w.base, 0);
        } else {
            cudaFree(w.base);
        }
    }
    cudaFree(w.lvl);
    cudaFree(w.b_stage);
    cudaFree(w.mst);
    cudaFree(w.hst);
    cudaFree(w.hrec);
    cudaFree(w.hflags);
    cudaFree(w.mflags);
    cudaFree(w.mrec);
    cudaFree(w.x_stage);
    cudaFree(w.bflag);
    if (w.s2) cudaStreamDestroy(w.s2);
    if (w.ev_a) cudaEventDestroy(w.ev_a);
    if (w.ev_b) cudaEventDestroy(w.ev_b);
    if (w.ev_done) cudaEventDestroy(w.ev_done);
    w = Workspace();
}

// Enqueue the plan kernels (AUTO threshold, per-block counts, one-CTA scan, task list) on stream
// s: the plan is built on the device from rowptr alone (sec.4.4's nnz-per-row pass, no level
// analysis); the host reads AnalyseOut afterwards.
int enqueue_plan(sptrsv_handle_s *h, cudaStream_t s) {
    const int32_t n = h->n;
    const int32_t ngroups = (n + 31) / 32;
    if (ngroups == 0) return SPTRSV_OK;
    const int nb = (ngroups + 1023) / 1024;
    const bool rev = h->tri & SPTRSV_TRI_UPPER;  // f4 upper: plan over logical (reversed) rows
    int32_t *bt = h->ws.blk, *bg = bt + nb, *off = bg + nb;
    k_auto_threshold<<<1, 1, 0, s>>>(h->ws.aout, n, h->threshold_user ? h->threshold : -1, h->subwarp_epl);
    k_plan_count<<<nb, 1024, 0, s>>>(h->rowptr, n, ngroups, h->mode, h->ws.aout, bt, bg, rev);
    k_plan_scan<<<1, 1024, 0, s>>>(bt, bg, nb, off, h->ws.aout);
    k_plan_write<<<nb, 1024, 0, s>>>(h->rowptr, n, ngroups, h->mode, h->ws.aout, off, h->ws.tasks, h->ws.task_w,
                                     rev);
    CK(cudaGetLastError());
    return SPTRSV_OK;
}

// the plan's shape from the read-back results
void adopt_plan(sptrsv_handle_s *h, const AnalyseOut &o) {
    const int32_t ngroups = (h->n + 31) / 32;
    h->threshold = o.threshold;
    h->dmin_log2 = o.med_log2;
    h->n_tasks = ngroups ? o.n_tasks : 0;
    h->n_thread_groups = ngroups ? o.n_tgroups : 0;
    h->n_sub_tasks = ngroups ? o.n_subtasks : 0;
    h->epl_eff = o.epl;
    // rows beyond thread level: warp rows are one task each, sub-warp tasks hold 32/W rows
    h->n_warp_rows = h->n_tasks - h->n_thread_groups - h->n_sub_tasks;
    h->plan = (h->n_thread_groups == ngroups) ? PLAN_THREAD
              : (h->n_thread_groups == 0 && h->n_sub_tasks == 0) ? PLAN_WARP : PLAN_LIST;
}

// Re-plan after a MODE / WARP_THRESHOLD change (synchronous: one D2H copy).
int build_plan(sptrsv_handle_s *h) {
    if (h->n == 0) return SPTRSV_OK;
    int rc = enqueue_plan(h, 0);
    if (rc) return rc;
    AnalyseOut o;
    CK(cudaMemcpy(&o, h->ws.aout, sizeof(o), cudaMemcpyDeviceToHost));
    adopt_plan(h, o);
    return SPTRSV_OK;
}

// discard.global.L2 over [p, p + bytes) (whole 128-B lines inside the range): drops a dead window's
// lines from L2 without write-back, which also ends their persisting status.
__global__ void k_l2_discard(char *p, size_t bytes) {
    const size_t lines = bytes / 128;
    for (size_t l = blockIdx.x * (size_t)blockDim.x + threadIdx.x; l < lines; l += (size_t)gridDim.x * blockDim.x)
        asm volatile("discard.global.L2 [%0], 128;" ::"l"(p + l * 128) : "memory");
}

// SolveState := 0 with the start ticket at gen << kGenShift (solve.cuh cta_ticket).  A kernel, not
// a host copy, so that a reset inside a stream capture is capturable.
__global__ void k_state_init(SolveState *st, uint32_t gen) {
    st->tk.v = (unsigned long long)gen << kGenShift;
}

int init_state(SolveState *st, uint32_t gen, cudaStream_t s) {
    CK(cudaMemsetAsync(st, 0, sizeof(SolveState), s));
    k_state_init<<<1, 1, 0, s>>>(st, gen);
    CK(cudaGetLastError());
    return SPTRSV_OK;
}


// a reset is due before the next launch: new configuration, epoch about to wrap, or the 40-bit
// ticket count of this generation about to overflow
bool reset_due(uint32_t since, unsigned grid) {
    return since >= kEpochResetAt || (unsigned long long)(since + 1) * grid >= (1ull << (kGenShift - 1));
}

}  // namespace

extern "C" {

int sptrsv_abi_version(void) { return SPTRSV_ABI_VERSION; }

const char *sptrsv_strerror(int status) {
    switch (status) {
        case SPTRSV_OK: return "ok";
        case SPTRSV_ERR_INVALID_ARG: return "invalid argument";
        case SPTRSV_ERR_NOT_LOWER: return "entry above the diagonal (column > row)";
        case SPTRSV_ERR_MISSING_DIAG: return "row without a diagonal as its last entry";
        case SPTRSV_ERR_ZERO_DIAG: return "zero diagonal";
        case SPTRSV_ERR_UNSORTED: return "columns not strictly increasing (unsorted or duplicate)";
        case SPTRSV_ERR_BAD_ROWPTR: return "malformed rowptr";
        case SPTRSV_ERR_BAD_COL: return "negative column index";
        case SPTRSV_ERR_TOO_LARGE: return "matrix too large for int32 CSR";
        case SPTRSV_ERR_CUDA: return "CUDA runtime error";
        case SPTRSV_ERR_ALLOC: return "allocation failed";
        case SPTRSV_ERR_TIMEOUT: return "watchdog timeout in solve";
        case SPTRSV_ERR_INEXACT:
            return "a chain quotient failed its exactness proof; the solve was aborted and the handle now proves "
                   "every quotient in-loop (re-solve)";
        case SPTRSV_ERR_STALE_LAUNCH:
            return "a captured solve was replayed after the handle's launch configuration changed (re-capture)";
        default: return "unknown status";
    }
}

int sptrsv_analyse_csr(int32_t n, const int32_t *rowptr, const int32_t *colidx, const double *val,
                       sptrsv_handle_t *out) {
    return sptrsv_analyse_csr_ex(n, rowptr, colidx, val, 0, out);
}

}  // extern "C"

namespace {
// block-diagonal concatenation (sptrsv_analyse_csr_batch): one system's rowptr shifted by the entries
// before it, its column indices by the rows before it (lower and upper alike: the blocks sit on the
// diagonal), its values copied
__global__ void k_concat_rowptr(const int32_t *__restrict__ src, int32_t n, int32_t row_off, int64_t nnz_off,
                                int32_t *__restrict__ dst) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) dst[row_off + i] = (int32_t)(src[i] + nnz_off);
}
__global__ void k_concat_colidx(const int32_t *__restrict__ src, int64_t nnz, int32_t row_off,
                                int32_t *__restrict__ dst) {
    const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < nnz) dst[j] = src[j] + row_off;
}
__global__ void k_set_i32(int32_t *p, int32_t v) { *p = v; }
}  // namespace

extern "C" {

int sptrsv_analyse_csr_batch(int32_t nsys, const int32_t *n, const int32_t *const *rowptr,
                             const int32_t *const *colidx, const double *const *val, int32_t tri_flags,
                             sptrsv_handle_t *out) {
    if (!out) return SPTRSV_ERR_INVALID_ARG;
    *out = nullptr;
    if (nsys < 1 || !n || !rowptr || !colidx || !val) return SPTRSV_ERR_INVALID_ARG;
    // each system's entry count: rowptr[n_s] (a rowptr[0] != 0 is caught by the validation below,
    // as a malformed rowptr of the concatenated system)
    std::vector<int64_t> nnz(nsys), z0(nsys + 1, 0);
    std::vector<int32_t> r0(nsys + 1, 0);
    for (int k = 0; k < nsys; ++k) {
        if (n[k] < 0 || !rowptr[k]) return SPTRSV_ERR_INVALID_ARG;
        int32_t last = 0, first = 0;
        if (cudaMemcpy(&last, rowptr[k] + n[k], sizeof(int32_t), cudaMemcpyDeviceToHost) != cudaSuccess ||
            cudaMemcpy(&first, rowptr[k], sizeof(int32_t), cudaMemcpyDeviceToHost) != cudaSuccess) {
            (void)cudaGetLastError();
            return SPTRSV_ERR_INVALID_ARG;
        }
        if (first != 0 || last < 0) return SPTRSV_ERR_BAD_ROWPTR;
        if (last > 0 && (!colidx[k] || (!val[k] && !(tri_flags & SPTRSV_TRI_UNIT_DIAG)))) return SPTRSV_ERR_INVALID_ARG;
        nnz[k] = last;
        if ((int64_t)r0[k] + n[k] > 0x7FFFFFFE) return SPTRSV_ERR_TOO_LARGE;
        r0[k + 1] = r0[k] + n[k];
        z0[k + 1] = z0[k] + last;
    }
    if (z0[nsys] > 0x7FFFFFFF) return SPTRSV_ERR_TOO_LARGE;
    const int32_t N = r0[nsys];
    const int64_t Z = z0[nsys];
    int32_t *rp = nullptr, *ci = nullptr;
    double *v = nullptr;
    auto fail = [&](int rc) {
        (void)cudaGetLastError();
        cudaFree(rp);
        cudaFree(ci);
        cudaFree(v);
        return rc;
    };
    if (cudaMalloc(&rp, sizeof(int32_t) * ((size_t)N + 1)) != cudaSuccess ||
        cudaMalloc(&ci, sizeof(int32_t) * (size_t)(Z > 0 ? Z : 1)) != cudaSuccess ||
        cudaMalloc(&v, sizeof(double) * (size_t)(Z > 0 ? Z : 1)) != cudaSuccess)
        return fail(SPTRSV_ERR_ALLOC);
    for (int k = 0; k < nsys; ++k) {
        if (n[k] > 0) k_concat_rowptr<<<(n[k] + 255) / 256, 256>>>(rowptr[k], n[k], r0[k], z0[k], rp);
        if (nnz[k] > 0) {
            k_concat_colidx<<<(unsigned)((nnz[k] + 255) / 256), 256>>>(colidx[k], nnz[k], r0[k], ci + z0[k]);
            if (val[k] && cudaMemcpyAsync(v + z0[k], val[k], sizeof(double) * (size_t)nnz[k], cudaMemcpyDeviceToDevice,
                                          0) != cudaSuccess)
                return fail(SPTRSV_ERR_CUDA);
        }
    }
    k_set_i32<<<1, 1>>>(rp + N, (int32_t)Z);
    if (cudaGetLastError() != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) return fail(SPTRSV_ERR_CUDA);
    sptrsv_handle_t h = nullptr;
    const int rc = sptrsv_analyse_csr_ex(N, rp, ci, (tri_flags & SPTRSV_TRI_UNIT_DIAG) && Z == 0 ? nullptr : v,
                                         tri_flags, &h);
    if (rc) return fail(rc);
    h->own_rowptr = rp;
    h->own_colidx = ci;
    h->own_val = v;
    *out = h;
    return SPTRSV_OK;
}

void size_l2_window(sptrsv_handle_s *h);


int sptrsv_analyse_csr_ex(int32_t n, const int32_t *rowptr, const int32_t *colidx, const double *val,
                          int32_t tri_flags, sptrsv_handle_t *out) {
    const auto t0 = std::chrono::steady_clock::now();
    if (!out) return SPTRSV_ERR_INVALID_ARG;
    *out = nullptr;
    if (n < 0 || (tri_flags & ~(SPTRSV_TRI_UPPER | SPTRSV_TRI_UNIT_DIAG))) return SPTRSV_ERR_INVALID_ARG;
    if (n > 0x7FFFFFFE) return SPTRSV_ERR_TOO_LARGE;
    // colidx / val may be NULL only when nnz == 0 (unit-diagonal identity), checked on the device
    if (!rowptr || (n > 0 && !(tri_flags & SPTRSV_TRI_UNIT_DIAG) && (!colidx || !val)))
        return SPTRSV_ERR_INVALID_ARG;
    int rc = set_kernel_attrs();
    if (rc) return rc;
    auto *h = new (std::nothrow) sptrsv_handle_s();
    if (!h) return SPTRSV_ERR_ALLOC;
    if (cudaGetDevice(&h->device) != cudaSuccess) {
        delete h;
        return SPTRSV_ERR_CUDA;
    }
    h->n = n;
    h->rowptr = rowptr;
    h->colidx = colidx;
    h->val = val;
    h->tri = tri_flags;
    // O(nnz) setup as ONE allocation, ONE memset, a fixed handful of kernels on the legacy stream
    // and ONE device->host copy of the results (Alg.5 l.1 "MALLOC(get_value, m)", PAPER.md:307;
    // "no preprocessing", :248): validation + in-degree + AUTO statistics (k_validate), the AUTO
    // warp threshold, the thread/warp plan (count, scan, write), the solve state.
    do {
        const size_t nn = (size_t)(n > 0 ? n : 1);
        const size_t ngroups = ((size_t)n + 31) / 32;
        const size_t nb = (ngroups + 1023) / 1024;
        auto al = [](size_t v) { return (v + 255) & ~(size_t)255; };
        const size_t o_rec = 0, o_flags = o_rec + al(16 * nn), o_indeg = o_flags + al(4 * nn),
                     o_tasks = o_indeg + al(4 * nn), o_tw = o_tasks + al(4 * nn), o_st = o_tw + al(nn),
                     o_out = o_st + al(sizeof(SolveState)), o_blk = o_out + al(sizeof(AnalyseOut)),
                     total = o_blk + al(4 * 3 * (nb ? nb : 1));
        cudaMemPool_t pool = ws_pool(h->device);
        if (pool && cudaMallocFromPoolAsync(&h->ws.base, total, pool, 0) == cudaSuccess) {
            h->ws.pooled = true;
        } else {
            (void)cudaGetLastError();
            h->ws.base = nullptr;
            if (cudaMalloc(&h->ws.base, total) != cudaSuccess) {
                rc = SPTRSV_ERR_ALLOC;
                break;
            }
        }
        char *b = static_cast<char *>(h->ws.base);
        h->ws.rec = reinterpret_cast<unsigned long long *>(b + o_rec);
        h->ws.flags = reinterpret_cast<uint32_t *>(b + o_flags);
        h->ws.indeg = reinterpret_cast<int32_t *>(b + o_indeg);
        h->ws.tasks = reinterpret_cast<int32_t *>(b + o_tasks);
        h->ws.task_w = reinterpret_cast<uint8_t *>(b + o_tw);
        h->ws.st = reinterpret_cast<SolveState *>(b + o_st);
        h->ws.aout = reinterpret_cast<AnalyseOut *>(b + o_out);
        h->ws.blk = reinterpret_cast<int32_t *>(b + o_blk);
        // everything zero (ready words: no epoch matches; counters; results), then status := ~0
        if (cudaMemsetAsync(h->ws.base, 0, total, 0) != cudaSuccess ||
            cudaMemsetAsync(&h->ws.aout->status, 0xff, sizeof(unsigned long long), 0) != cudaSuccess) {
            rc = SPTRSV_ERR_CUDA;
            break;
        }
        if (n > 0) {
            k_validate<<<(n + 255) / 256, 256>>>(rowptr, colidx, val, n, h->ws.indeg, h->ws.aout, tri_flags);
            k_grid_probe<<<1, 32>>>(rowptr, colidx, n, h->ws.aout, tri_flags);
            k_grid_check<<<(n + 255) / 256, 256>>>(rowptr, colidx, n, h->ws.aout, tri_flags);
            if (cudaGetLastError() != cudaSuccess) {
                rc = SPTRSV_ERR_CUDA;
                break;
            }
            rc = enqueue_plan(h, 0);
            if (rc) break;
        }
        h->gen = 1;
        rc = init_state(h->ws.st, h->gen, 0);
        if (rc) break;
        AnalyseOut o;
        if (cudaMemcpy(&o, h->ws.aout, sizeof(o), cudaMemcpyDeviceToHost) != cudaSuccess) {
            rc = SPTRSV_ERR_CUDA;
            break;
        }
        if (o.status != ~0ull) {
            rc = -(int)(o.status & 0xff);
            break;
        }
        h->nnz = n > 0 ? o.nnz : 0;
        h->max_row = o.max_row;
        h->near_deps = (int64_t)(o.near & 0xFFFFFFFFull);
        h->warp_deps = (int64_t)(o.near >> 32);
        h->prev_deps = (int64_t)(o.prev & 0xFFFFFFFFull);
        h->mid_breaks = o.mid_breaks;
        h->near_rows = (int64_t)(o.prev >> 32);
        h->grid_m = n > 0 ? o.grid_m : 0;
        h->grid_viol = o.grid_viol;
        h->grid_fast = o.grid_fast;
        h->grid_far = o.grid_far;
        if (n > 0) adopt_plan(h, o);
        else h->plan = PLAN_THREAD;
        h->since_reset = 0;
    } while (0);
    if (rc != SPTRSV_OK) {
        (void)cudaGetLastError();
        free_ws(h->ws);
        delete h;
        return rc;
    }
    size_l2_window(h);
    h->analyse_ms =
        std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
    *out = h;
    return SPTRSV_OK;
}

namespace {

// One solve launch: which kernel, its geometry, and how it is parameterised.  plan_launch is the
// single source of truth: sptrsv_get_info, sptrsv_solve_host's transfer overlap and the epoch
// arithmetic all read the engine / geometry it actually picked.
struct Launch {
    const void *fn = nullptr;
    dim3 grid, block;
    size_t smem = 0;
    int key = 0;      // configuration identity (the epoch arithmetic needs a fixed grid per key)
    int engine = 0;   // engine launched (ENG_*; 30 + v for the paper's Alg. v)
    int cta = 0;      // threads per CTA
    int K = 1;        // thread-level rows per lane
    bool coop = false;  // cooperative launch (every CTA co-resident: LEANP's static work assignment)
};

// Size the device's persisting L2 set-aside for the handle's ready-word window (SPTRSV_OPT_L2_WINDOW):
// grown to the window (up to persistingL2CacheMaxSize); l2_hit = 1 if it holds the whole window,
// -1 (no window) otherwise -- a partial window (c3's 67 MB of records) left the time unchanged and
// added DRAM traffic (361.6 vs 314.6 MB per launch).  Host-only, synchronous: called from analyse
// and set_option so that a first solve inside a stream capture never changes device limits.  The
// limit the library found is remembered per device and restored by the last handle's destroy.
void size_l2_window(sptrsv_handle_s *h) {
    h->l2_hit = -1.f;
    if (!h->l2_window || h->n == 0) {
        l2_limit_release(h);
        return;
    }
    const size_t wbytes = (h->proto == PROTO_FLAGS ? sizeof(uint32_t) : 16) * (size_t)h->n;
    int maxp = 0;
    size_t cur = 0;
    {
        std::lock_guard<std::mutex> lk(g_l2_mu);
        L2Limit &e = g_l2[h->device & 255];
        if (cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, h->device) == cudaSuccess &&
            cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize) == cudaSuccess) {
            if (e.users == 0) e.orig = cur;  // the value found before any windowed handle
            const size_t want = std::min(wbytes, (size_t)maxp);
            if (cur < want && cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want) == cudaSuccess) cur = want;
            h->l2_hit = cur >= wbytes ? 1.f : -1.f;
            if (h->l2_hit > 0.f && !h->l2_user) {
                h->l2_user = true;
                e.users++;
            }
            if (e.users == 0 && cur != e.orig) (void)cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, e.orig);
        }
        (void)cudaGetLastError();
    }
    if (h->l2_hit <= 0.f) l2_limit_release(h);
}

// ENGINE_AUTO, from analyse's O(nnz) statistics:
//   near-dependency systems that are not pure chains, <= kSmallAutoN rows, fitting one CTA's
//   shared memory (c1, small grids)                              -> SMALL (any plan, any form)
//   plans with warp-level rows                                   -> HYBRID
//   all-thread plans, < 1/4 of the rows waiting on a row < 256 away -> LEAN
//   all-thread plans, >= 1/4 of the dependencies on row i-1 (chains, grids) -> CHAIN
//   other near-dependency plans (small levels, c1)               -> ONE-SHOT (in-CTA smem copy of x)
// f4 (upper / unit) handles: HYBRID for warp rows, else CHAIN (chains) or LEAN.
bool small_fits(const sptrsv_handle_s *h) {
    return h->n > 0 && h->n <= (1 << 20) && small_smem_bytes(h->n, h->nnz) <= kSmallSmemMax;
}

// ENGINE_GRID (solve_grid.cuh): usable when analyse found a line length m under which every row
// keeps the band order (any triangular form, in logical rows); AUTO takes it for 2D grid-shaped factors -- m >= 32
// columns, >= 32 lines, >= 1/2 of the off-diagonals north / west neighbours, >= 1/4 west (the
// wavefront runs along the lines), <= 1/8 far entries.
bool grid_ok(const sptrsv_handle_s *h) {
    const long long offdiag = (h->tri & 2) ? h->nnz : h->nnz - h->n;  // unit handles store no diagonal
    return h->n > 0 && h->grid_m >= 2 && h->grid_viol == 0 && offdiag > 0;
}
bool grid_auto(const sptrsv_handle_s *h) {
    if (!grid_ok(h) || h->proto != PROTO_FUSED) return false;
    const long long offdiag = (h->tri & 2) ? h->nnz : h->nnz - h->n;
    const long long lines = ((long long)h->n + h->grid_m - 1) / h->grid_m;
    // ... and no (or few) far entries: a 3D grid's wavefront is far shorter than its line count (levels
    // ~ nx + ny + nz, lines ny * nz), so the level-parallel engines win there (64x48x20: ONE-SHOT 145 us,
    // GRID 283 us; 128^3: CHAIN 1.8 ms, GRID 4.5 ms), while 2D grids are GRID's (100^2: 57 vs 142 us)
    return h->grid_m >= 32 && lines >= 32 && 2 * h->grid_fast >= offdiag && 4 * h->prev_deps >= offdiag &&
           8 * h->grid_far <= offdiag;
}

int resolve_engine(const sptrsv_handle_s *h) {
    if (h->engine == ENG_SMALL && small_fits(h)) return ENG_SMALL;
    if (h->engine == ENG_GRID && grid_ok(h)) return ENG_GRID;
    const long long offdiag = (h->tri & 2) ? h->nnz : h->nnz - h->n;  // unit handles store no diagonal
    // chains: >= 1/4 of the dependencies on the previous row AND runs of such rows long enough for
    // CHAIN's in-warp steps to pay (mean run n / (rows without one) >= 64 rows, one CHAIN warp): with
    // short runs CHAIN serialises its warps through every run that crosses a warp boundary (c2i,
    // runs of 10: 11.5 ms on CHAIN, 74 us on LEAN)
    // ... and runs that CHAIN's warps can take whole: CHAIN solves a warp's 64 rows in row order, so a
    // run starting inside a warp waits for the previous run's tail -- on grids whose side is not a
    // multiple of 64 that serialises whole grid lines (1000^2 grid: 94 ms on CHAIN, 2.9 ms on
    // ONE-SHOT; 500^2: 24.6 vs 0.84 ms on LEAN).  Mean run >= 2048 rows (1024^2 grid: LEANP 1.73 ms
    // beats CHAIN's 2.33; 2048^2: CHAIN 5.1 ms, the rest >= 13 ms) and <= 1 run start per 4096 rows
    // off a warp boundary.
    const bool chains = offdiag > 0 && 4 * h->prev_deps >= offdiag &&
                        2048 * ((int64_t)h->n - h->prev_deps) <= (int64_t)h->n && 4096 * h->mid_breaks <= (int64_t)h->n;
    const bool near = offdiag > 0 && 4 * h->near_rows >= (int64_t)h->n;
    // a pure chain: almost every row waits on its predecessor and little else (critical path ~ n rows;
    // CHAIN's in-register hop beats SMALL's shared-memory pass there: 1024-row chain 111 vs 200 us)
    const bool pure_chain = 10 * h->prev_deps >= 9 * (int64_t)h->n && 4 * offdiag <= 5 * (int64_t)h->n;
    // AUTO: small near-dependency systems that fit one CTA (c1, small grids, short dense-ish rows) ->
    // SMALL, whatever the plan (measured: c1 18 vs 29 us ONE-SHOT, 32x32 grid 22 vs 169 us CHAIN,
    // 600 rows x 20 entries 38 vs 99 us)
    // (not when the user asked for warp-level rows: MODE 2 / 3 plans keep their warp engine)
    if (h->engine == ENG_AUTO && h->mode <= 1 && near && !pure_chain && h->n <= kSmallAutoN && small_fits(h))
        return ENG_SMALL;
    if (h->engine == ENG_AUTO && h->mode <= 1 && grid_auto(h)) return ENG_GRID;
    if (h->plan != PLAN_THREAD)  // ONE-SHOT has no sub-warp rows
        return (h->engine == ENG_ONESHOT && !h->tri && h->n_sub_tasks == 0) ? ENG_ONESHOT : ENG_HYBRID;
    if (h->engine != ENG_AUTO) return (h->tri && h->engine == ENG_ONESHOT) ? ENG_LEAN : h->engine;
    const int lean_auto = h->no_coop ? ENG_LEAN : ENG_LEANP;  // LEANP needs a cooperative launch
    if (h->tri) return chains ? ENG_CHAIN : lean_auto;
    if (offdiag <= 0 || 4 * h->near_rows < (int64_t)h->n) return lean_auto;
    return chains ? ENG_CHAIN : ENG_ONESHOT;
}

typedef void (*lean_fn)(SolveParams);

// LEAN for lower thread-level plans: CTA size ct in {128, 256, 512} (0 = 256) and the
// register budget occ = resident 256-thread CTAs per SM targeted (5..8), i.e.
// __launch_bounds__(ct, occ * 256 / ct).  Returns nullptr for an unsupported pair.
#define LEAN_OCC(CT_, M5, M6, M7, M8)                                                               \
    {{k_solve_lean<PROTO_FLAGS, M5, false, false, CT_>, k_solve_lean<PROTO_FUSED, M5, false, false, CT_>}, \
     {k_solve_lean<PROTO_FLAGS, M6, false, false, CT_>, k_solve_lean<PROTO_FUSED, M6, false, false, CT_>}, \
     {k_solve_lean<PROTO_FLAGS, M7, false, false, CT_>, k_solve_lean<PROTO_FUSED, M7, false, false, CT_>}, \
     {k_solve_lean<PROTO_FLAGS, M8, false, false, CT_>, k_solve_lean<PROTO_FUSED, M8, false, false, CT_>}}
lean_fn lean_lower_kernel(int proto, int occ, int ct) {
    static const lean_fn tab[3][4][2] = {LEAN_OCC(128, 10, 12, 14, 16), LEAN_OCC(256, 5, 6, 7, 8),
                                         LEAN_OCC(512, 2, 3, 3, 4)};
    const int c = ct == 128 ? 0 : ct == 256 ? 1 : 2;
    if (occ < 5 || occ > 8) return nullptr;
    return tab[c][occ - 5][proto ? 1 : 0];
}
#undef LEAN_OCC

lean_fn lean_tri_kernel(int proto, int tri) {
    static const lean_fn tab[4][2] = {
        {k_solve_lean<PROTO_FLAGS, 5>, k_solve_lean<PROTO_FUSED, 5>},
        {k_solve_lean<PROTO_FLAGS, 5, true, false>, k_solve_lean<PROTO_FUSED, 5, true, false>},
        {k_solve_lean<PROTO_FLAGS, 5, false, true>, k_solve_lean<PROTO_FUSED, 5, false, true>},
        {k_solve_lean<PROTO_FLAGS, 5, true, true>, k_solve_lean<PROTO_FUSED, 5, true, true>},
    };
    return tab[tri & 3][proto ? 1 : 0];
}

lean_fn tri_warp_kernel(int proto, int tri, int plan, int ct) {
#define TRI_ROW(U, N, C)                                                                                 \
    {k_solve_tri_warp<PROTO_FLAGS, U, N, PLAN_WARP, C>, k_solve_tri_warp<PROTO_FUSED, U, N, PLAN_WARP, C>, \
     k_solve_tri_warp<PROTO_FLAGS, U, N, PLAN_LIST, C>, k_solve_tri_warp<PROTO_FUSED, U, N, PLAN_LIST, C>}
    static const lean_fn tab[2][4][4] = {
        {TRI_ROW(false, false, 64), TRI_ROW(true, false, 64), TRI_ROW(false, true, 64), TRI_ROW(true, true, 64)},
        {TRI_ROW(false, false, 256), TRI_ROW(true, false, 256), TRI_ROW(false, true, 256),
         TRI_ROW(true, true, 256)}};
#undef TRI_ROW
    return tab[ct == 256 ? 1 : 0][tri & 3][(plan == PLAN_LIST ? 2 : 0) + (proto ? 1 : 0)];
}

lean_fn chain_kernel(int proto, int tri, int K, bool safe) {
#define CHAIN_ROW(U_, N_, S_)                                                                          \
    {{k_solve_chain<PROTO_FLAGS, 1, U_, N_, S_>, k_solve_chain<PROTO_FUSED, 1, U_, N_, S_>},           \
     {k_solve_chain<PROTO_FLAGS, 2, U_, N_, S_>, k_solve_chain<PROTO_FUSED, 2, U_, N_, S_>}}
    static const lean_fn tab[2][4][2][2] = {
        {CHAIN_ROW(false, false, false), CHAIN_ROW(true, false, false), CHAIN_ROW(false, true, false),
         CHAIN_ROW(true, true, false)},
        {CHAIN_ROW(false, false, true), CHAIN_ROW(true, false, true), CHAIN_ROW(false, true, true),
         CHAIN_ROW(true, true, true)}};
#undef CHAIN_ROW
    return tab[safe ? 1 : 0][tri & 3][K - 1][proto ? 1 : 0];
}

int plan_launch(sptrsv_handle_s *h, Launch *L) {
    if (h->variant) {  // the paper's kernels, control flow as printed (solve_paper.cuh; ablation only)
        L->block = dim3(kPaperCta);
        if (h->variant == 3) {
            L->fn = (const void *)k_paper_alg3;
            L->grid = dim3((unsigned)((h->n + kPaperCta / 32 - 1) / (kPaperCta / 32)));
        } else {
            L->fn = h->variant == 4 ? (const void *)k_paper_alg4 : (const void *)k_paper_alg5;
            L->grid = dim3((unsigned)((h->n + kPaperCta - 1) / kPaperCta));
        }
        L->engine = 30 + h->variant;
        L->cta = kPaperCta;
        L->key = (6000000 + h->variant * 100000) ^ (int)L->grid.x * 7919;
        return SPTRSV_OK;
    }
    const int engine = resolve_engine(h);
    const int user = h->cta_threads;
    L->engine = engine;
    if (engine == ENG_SMALL) {  // one CTA, the system in shared memory (solve_small.cuh)
        static const lean_fn tab[4] = {k_solve_small<false, false>, k_solve_small<true, false>,
                                       k_solve_small<false, true>, k_solve_small<true, true>};
        // the dynamic shared memory limit is raised to what this launch needs (per device: the attribute
        // is per context), not to the 226 KB maximum
        static int attr_set[64][4] = {};
        const int t = h->tri & 3, dv = h->device & 63;
        const size_t need = small_smem_bytes(h->n, h->nnz);
        L->fn = (const void *)tab[t];
        if ((size_t)attr_set[dv][t] < need) {
            if (cudaFuncSetAttribute(L->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)need) != cudaSuccess) {
                (void)cudaGetLastError();
                return SPTRSV_ERR_CUDA;
            }
            attr_set[dv][t] = (int)need;
        }
        // 256 threads (default): measured best on c1 / 32x32 grids (fewer spinning warps leave the
        // issue slots to the ones on the critical path; 1024 threads: c1 32.8 us, 256: 18.5 us)
        const int rows32 = (int)std::min<long long>(kSmallCtaMax, ((long long)h->n + 31) / 32 * 32);
        int ct = std::min(kSmallCta, rows32);
        if (user >= 32 && user <= kSmallCtaMax && user % 32 == 0) ct = std::min(user, rows32);
        L->cta = ct;
        L->grid = dim3(1u);
        L->block = dim3((unsigned)ct);
        L->smem = small_smem_bytes(h->n, h->nnz);
        L->key = (9000000 + h->tri * 10000 + ct) ^ h->n * 7919;
        return SPTRSV_OK;
    }
    if (engine == ENG_HYBRID) {  // warp-level rows: one task per warp (solve_tri.cuh), any triangular form
        if (h->plan == PLAN_THREAD) {  // HYBRID forced on an all-thread plan: run it as LEAN
            L->engine = ENG_LEAN;
        } else {
            const int ct = user == 256 ? 256 : kTriWarpCta;  // 64 (default) or 256 threads
            L->fn = (const void *)tri_warp_kernel(h->proto, h->tri, h->plan, ct);
#ifdef SPTRSV_MEASURE_HYBRID_SMEM  // measurement builds only (tools/): cap residency with padding
            L->smem = SPTRSV_MEASURE_HYBRID_SMEM;
            if (cudaFuncSetAttribute(L->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L->smem) != cudaSuccess)
                return SPTRSV_ERR_CUDA;
#endif
            L->cta = ct;
            L->grid = dim3((unsigned)((h->n_tasks + ct / 32 - 1) / (ct / 32)));
            L->block = dim3((unsigned)ct);
            L->key = (7500000 + h->proto * 100000 + h->tri * 10000 + h->plan * 1000 + ct / 64) ^ (int)L->grid.x * 7919;
            return SPTRSV_OK;
        }
    }
    if (engine == ENG_GRID) {  // wavefront bands of 32 columns, one CTA per band (solve_grid.cuh)
#define GRID_ROW(F_, U_, N_)                                                                               \
    {{k_solve_grid<PROTO_FLAGS, false, F_, U_, N_>, k_solve_grid<PROTO_FUSED, false, F_, U_, N_>},            \
     {k_solve_grid<PROTO_FLAGS, true, F_, U_, N_>, k_solve_grid<PROTO_FUSED, true, F_, U_, N_>}}
        static const lean_fn tab[2][4][2][2] = {
            {GRID_ROW(false, false, false), GRID_ROW(false, true, false), GRID_ROW(false, false, true),
             GRID_ROW(false, true, true)},
            {GRID_ROW(true, false, false), GRID_ROW(true, true, false), GRID_ROW(true, false, true),
             GRID_ROW(true, true, true)}};
#undef GRID_ROW
        const int fv = h->grid_far > 0 ? 1 : 0;
        L->fn = (const void *)tab[fv][h->tri & 3][h->chain_div == 1 ? 1 : 0][h->proto ? 1 : 0];
        L->smem = grid_smem_bytes(32 * std::max(1, h->max_row));
        static size_t attr_set[64][32] = {};  // per device and kernel: the dynamic smem limit raised so far
        size_t &cur = attr_set[h->device & 63][fv * 16 + (h->tri & 3) * 4 + (h->chain_div == 1 ? 2 : 0) + (h->proto ? 1 : 0)];
        if (cur < L->smem) {
            if (cudaFuncSetAttribute(L->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L->smem) != cudaSuccess) {
                (void)cudaGetLastError();
                return SPTRSV_ERR_CUDA;
            }
            cur = L->smem;
        }
        L->cta = 32 * kGridWarps;
        L->grid = dim3((unsigned)((h->grid_m + 31) / 32));
        L->block = dim3((unsigned)L->cta);
        L->key = (10000000 + h->proto * 100000 + (h->chain_div == 1 ? 500 : 0)) ^ (int)L->grid.x * 7919;
        return SPTRSV_OK;
    }
    if (L->engine == ENG_CHAIN) {  // warp-sequential in-warp chains (solve_chain.cuh): 64..256 threads
        const int K = h->rows_per_lane == 1 ? 1 : 2;  // other values: the default 2
        const int cta = (user == 64 || user == 128 || user == 256) ? user : kChainCta;
        const int warps = cta / 32;
        const long long rows_per_cta = (long long)warps * 32 * K;
        L->fn = (const void *)chain_kernel(h->proto, h->tri, K, h->chain_div == 1);
        L->cta = cta;
        L->K = K;
        L->grid = dim3((unsigned)((h->n + rows_per_cta - 1) / rows_per_cta));
        L->block = dim3((unsigned)cta);
        L->smem = (size_t)warps * chain_warp_smem_bytes(K);
        if (L->smem > 48 * 1024 &&
            cudaFuncSetAttribute(L->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L->smem) != cudaSuccess) {
            (void)cudaGetLastError();
            return SPTRSV_ERR_CUDA;
        }
        L->key = (8000000 + h->proto * 100000 + K * 10000 + h->tri * 1000 + cta + (h->chain_div == 1 ? 500 : 0)) ^
                 (int)L->grid.x * 7919;
        return SPTRSV_OK;
    }
    if (L->engine == ENG_LEANP) {  // persistent pipelined LEAN (solve_lean.cuh), experimental
#ifndef SPTRSV_LEANP_MINB
#define SPTRSV_LEANP_MINB 3
#endif
        constexpr int MB = SPTRSV_LEANP_MINB;
        static const lean_fn tab[4][2] = {
            {k_solve_leanp<PROTO_FLAGS, MB>, k_solve_leanp<PROTO_FUSED, MB>},
            {k_solve_leanp<PROTO_FLAGS, MB, true, false>, k_solve_leanp<PROTO_FUSED, MB, true, false>},
            {k_solve_leanp<PROTO_FLAGS, MB, false, true>, k_solve_leanp<PROTO_FUSED, MB, false, true>},
            {k_solve_leanp<PROTO_FLAGS, MB, true, true>, k_solve_leanp<PROTO_FUSED, MB, true, true>}};
        L->fn = (const void *)tab[h->tri & 3][h->proto ? 1 : 0];
        int per_sm = 0, sms = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, L->fn, kLeanCta, 0) != cudaSuccess ||
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->device) != cudaSuccess || per_sm < 1) {
            (void)cudaGetLastError();
            return SPTRSV_ERR_CUDA;
        }
        const long long nblk = ((long long)h->n + kLeanCta - 1) / kLeanCta;
#ifdef SPTRSV_MEASURE_LEANP_PER_SM  // measurement builds only: fewer resident CTAs than fit
        per_sm = std::min(per_sm, SPTRSV_MEASURE_LEANP_PER_SM);
#endif
        const long long g = std::min<long long>(nblk, (long long)per_sm * sms);
        L->cta = kLeanCta;
        L->grid = dim3((unsigned)g);
        L->block = dim3((unsigned)kLeanCta);
        L->coop = true;
        L->key = (9500000 + h->proto * 100000 + h->tri * 10) ^ (int)L->grid.x * 7919;
        return SPTRSV_OK;
    }
    if (L->engine == ENG_LEAN) {  // minimal one-shot kernel for all-thread-level plans (solve_lean.cuh)
        int ct = kLeanCta;
        if (h->tri) {
            L->fn = (const void *)lean_tri_kernel(h->proto, h->tri);
        } else {
            // CTA size 128 / 256 (default) / 512 (option CTA_THREADS) and the register budget
            // (option LEAN_OCCUPANCY = resident 256-thread CTAs per SM it targets: 5..8)
            if (user == 128 || user == 512) ct = user;
            L->fn = (const void *)lean_lower_kernel(h->proto, h->lean_minb, ct);
            if (!L->fn) return SPTRSV_ERR_INVALID_ARG;
        }
        L->cta = ct;
        L->grid = dim3((unsigned)((h->n + ct - 1) / ct));
        L->block = dim3((unsigned)ct);
        L->key = (5000000 + h->proto * 100000 + h->lean_minb * 1000 + h->tri * 10 + ct / 128) ^ (int)L->grid.x * 7919;
        return SPTRSV_OK;
    }
    // ONE-SHOT (solve.cuh k_solve), lower handles only: staged CSR slices and an in-CTA shared-memory copy of
    // x.  64-thread CTAs on plans with warp-level rows; 1024 for small (n <= 32768) thread-level systems
    // (more dependencies resolved in-CTA: c1 29.7 -> 26.7 us); else 256.
    int cta = h->plan != PLAN_THREAD ? 64 : h->n <= 32768 ? 1024 : 256;
    if (user >= 64) cta = user;  // (32: SMALL only)
    const int warps = cta / 32;
    L->engine = ENG_ONESHOT;
    L->fn = (const void *)solve_kernel(h->plan, h->proto);
    L->cta = cta;
    L->grid = dim3((unsigned)((h->n_tasks + warps - 1) / warps));
    L->block = dim3((unsigned)cta);
    L->smem = solve_smem_bytes(cta, h->stage && h->plan != PLAN_WARP);
    L->key = (4000000 + (h->plan * 2 + h->proto) * 100000 + cta) ^ (int)L->grid.x * 7919;
    return SPTRSV_OK;
}

}  // namespace

static int solve_impl(sptrsv_handle_t h, const double *b, double *x, double *x_host, sptrsv_stream_t stream,
                      const uint32_t *bflag = nullptr, uint32_t bseq = 0, int bshift = kBChunkShift,
                      bool host_state = false);

int sptrsv_solve(sptrsv_handle_t h, const double *b, double *x, sptrsv_stream_t stream) {
    return solve_impl(h, b, x, nullptr, stream);
}

// x_host (LEAN only, from sptrsv_solve_host): device-mapped pinned host copy target of x
static int solve_impl(sptrsv_handle_t h, const double *b, double *x, double *x_host, sptrsv_stream_t stream,
                      const uint32_t *bflag, uint32_t bseq, int bshift, bool host_state) {
    if (!h) return SPTRSV_ERR_INVALID_ARG;
    if (h->n == 0) return SPTRSV_OK;
    if (!b || !x || b == x) return SPTRSV_ERR_INVALID_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess || cur != h->device) {
        (void)cudaGetLastError();
        return SPTRSV_ERR_INVALID_ARG;  // the handle's device must be current (its stream, its workspace)
    }
    Launch L;
    int rc = plan_launch(h, &L);
    if (rc) return rc;
    // host_state (sptrsv_solve_host on a LEANP plan): the LEAN kernel on the host-path state set
    host_state = host_state && L.engine == ENG_LEANP;
    if (host_state) {
        const int saved = h->engine;
        h->engine = ENG_LEAN;
        L = Launch();
        rc = plan_launch(h, &L);
        h->engine = saved;
        if (rc) return rc;
        Workspace &w = h->ws;
        if (!w.hst) {
            const size_t nn = (size_t)(h->n > 0 ? h->n : 1);
            if (cudaMalloc(&w.hst, sizeof(SolveState)) != cudaSuccess || cudaMalloc(&w.hrec, 16 * nn) != cudaSuccess ||
                cudaMalloc(&w.hflags, 4 * nn) != cudaSuccess) {
                (void)cudaGetLastError();
                cudaFree(w.hst);
                cudaFree(w.hrec);
                cudaFree(w.hflags);
                w.hst = nullptr, w.hrec = nullptr, w.hflags = nullptr;
                return SPTRSV_ERR_ALLOC;
            }
            h->hlaunch_key = -1;
        }
    }
    SolveState *st = host_state ? h->ws.hst : h->ws.st;
    unsigned long long *rec = host_state ? h->ws.hrec : h->ws.rec;
    uint32_t *flags = host_state ? h->ws.hflags : h->ws.flags;
    int &launch_key = host_state ? h->hlaunch_key : h->launch_key;
    uint32_t &since_reset = host_state ? h->hsince_reset : h->since_reset;
    uint32_t &gen = host_state ? h->hgen : h->gen;
    // The epoch of a solve is derived on the device from the start ticket and the
    // grid size (solve.cuh SolveState); a new launch configuration, or an epoch
    // about to wrap, re-zeroes the flags / records and the counters first.
    if (L.key != launch_key || reset_due(since_reset, L.grid.x)) {
        const size_t nn = (size_t)(h->n > 0 ? h->n : 1);
        CK(cudaMemsetAsync(flags, 0, sizeof(uint32_t) * nn, s));
        CK(cudaMemsetAsync(rec, 0, 16 * nn, s));
        gen = (gen + 1) & 0xFFFFFFu;
        since_reset = 0;
        rc = init_state(st, gen, s);
        if (rc) return rc;
        launch_key = L.key;
    }
    SolveParams p{};
    p.rowptr = h->rowptr;
    p.colidx = h->colidx;
    p.val = h->val;
    p.b = b;
    p.x = x;
    p.flags = flags;
    p.rec = rec;
    p.tasks = h->ws.tasks;
    p.task_w = h->ws.task_w;
    p.st = st;
    p.nnz = h->nnz;
    p.n = h->n;
    p.n_tasks = h->n_tasks;
    p.epoch0 = 1;
    p.gen = gen;
    p.grid = L.grid.x;
    p.backoff_min = h->backoff_min;
    p.backoff_max = h->backoff_max;
    p.spin_limit = h->spin_limit;
    p.stage = h->stage;
    p.local = h->local;
    p.poll_gap = h->poll_gap;
    p.poll_one = h->poll_one;
    p.split_last = h->split_last;
    p.chain_div = h->chain_div;
    p.grid_m = h->grid_m;
    p.grid_lines = h->grid_m > 0 ? (int32_t)(((long long)h->n + h->grid_m - 1) / h->grid_m) : 0;  // (upper: n % m == 0)
    p.grid_ecap = 32 * std::max(1, h->max_row);
    p.grid_far = h->grid_far > 0 ? 1 : 0;
    p.x_host = x_host;
    p.bflag = bflag;
    p.bseq = bseq;
    p.bshift = bshift;
    p.trace = h->trace;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = L.grid;
    cfg.blockDim = L.block;
    cfg.dynamicSmemBytes = L.smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[2];
    cfg.numAttrs = 0;
    if (L.coop) {
        cudaLaunchAttribute &a = attr[cfg.numAttrs++];
        a.id = cudaLaunchAttributeCooperative;
        a.val.cooperative = 1;
    }
    cfg.attrs = attr;
    // The ready words (FLAGS: flags, FUSED: records) in a persisting L2 window -- north_star's
    // "L2 access-policy window pinning the flags".  They are the handle's workspace, re-read by
    // every dependent row and re-written every solve; persisting lines are not evicted by the
    // streamed CSR nor by other traffic between solves (bench.py's 256 MiB flush included), so
    // polls of not-yet-published dependencies and the publishes hit L2 (c2 41.0 -> 32.8 us).
    // The device's persisting set-aside is grown to the window (size_l2_window, at analyse time and
    // on option changes -- never inside a stream capture); a window it cannot hold whole is not used.
    void *wbase = host_state ? nullptr : h->proto == PROTO_FLAGS ? (void *)h->ws.flags : (void *)h->ws.rec;
    const size_t wbytes = (h->proto == PROTO_FLAGS ? sizeof(uint32_t) : 16) * (size_t)h->n;
    if (h->l2_window && wbase && h->l2_hit == 0.f) size_l2_window(h);  // normally done at analyse / set_option
    if (h->l2_window && wbase && h->l2_hit > 0.f) {
        cudaLaunchAttribute &a = attr[cfg.numAttrs++];
        a.id = cudaLaunchAttributeAccessPolicyWindow;
        a.val.accessPolicyWindow.base_ptr = wbase;
        a.val.accessPolicyWindow.num_bytes = std::min(wbytes, (size_t)0x7FFFFFFF);
        a.val.accessPolicyWindow.hitRatio = h->l2_hit;
        a.val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        a.val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    }
    const cudaError_t e = cudaLaunchKernelEx(&cfg, (void (*)(SolveParams))L.fn, p);
    if (e != cudaSuccess) {
        (void)cudaGetLastError();
        if (L.coop && h->engine == ENG_AUTO && !h->no_coop) {
            // the device would not co-schedule the persistent grid (another process holds SMs, MPS
            // limits ...): AUTO falls back to the non-persistent LEAN for this handle from now on
            h->no_coop = true;
            return solve_impl(h, b, x, x_host, stream, bflag, bseq, bshift, host_state);
        }
        return SPTRSV_ERR_CUDA;
    }
    h->solves++;
    since_reset++;
    return SPTRSV_OK;
}

namespace {
__global__ void k_col_gather(const double *__restrict__ B, int64_t ldb, double *__restrict__ b, int32_t n) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) b[i] = B[(size_t)i * ldb];
}
__global__ void k_col_scatter(const double *__restrict__ x, double *__restrict__ X, int64_t ldx, int32_t n) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) X[(size_t)i * ldx] = x[i];
}
}  // namespace

int sptrsv_solve_multi(sptrsv_handle_t h, const double *B, double *X, int32_t nrhs, int64_t ldb, int64_t ldx,
                       sptrsv_stream_t stream) {
    if (!h) return SPTRSV_ERR_INVALID_ARG;
    if (nrhs < 1 || nrhs > 32 || ldb < nrhs || ldx < nrhs) return SPTRSV_ERR_INVALID_ARG;
    if (h->n == 0) return SPTRSV_OK;
    if (!B || !X || (const double *)X == B) return SPTRSV_ERR_INVALID_ARG;
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess || cur != h->device) {
        (void)cudaGetLastError();
        return SPTRSV_ERR_INVALID_ARG;
    }
    cudaStream_t s = (cudaStream_t)stream;
    Launch L0;
    int rc0 = plan_launch(h, &L0);
    if (rc0) return rc0;
    if (h->tri || L0.engine == ENG_CHAIN) {
        // Column by column through the handle's own engine: f4 (upper / unit) handles, and plans
        // that run CHAIN, whose in-register chains are worth more than k_solve_multi's one hop per
        // row for all columns (c3, 8 columns: 77 ms in k_solve_multi, 8 x 5 ms here).  Each column
        // is gathered into contiguous staging, solved, and scattered back, all on `stream`.
        const size_t bytes = sizeof(double) * (size_t)h->n;
        if (!h->ws.b_stage && cudaMalloc(&h->ws.b_stage, bytes) != cudaSuccess) {
            (void)cudaGetLastError();
            return SPTRSV_ERR_ALLOC;
        }
        if (!h->ws.x_stage && cudaMalloc(&h->ws.x_stage, bytes) != cudaSuccess) {
            (void)cudaGetLastError();
            return SPTRSV_ERR_ALLOC;
        }
        const unsigned g = (unsigned)((h->n + 255) / 256);
        for (int r = 0; r < nrhs; ++r) {
            k_col_gather<<<g, 256, 0, s>>>(B + r, ldb, h->ws.b_stage, h->n);
            CK(cudaGetLastError());
            int rc = solve_impl(h, h->ws.b_stage, h->ws.x_stage, nullptr, stream);
            if (rc) return rc;
            k_col_scatter<<<g, 256, 0, s>>>(h->ws.x_stage, X + r, ldx, h->n);
            CK(cudaGetLastError());
        }
        return SPTRSV_OK;
    }
    const size_t words = (size_t)h->n * (size_t)nrhs;
    if (nrhs > h->ws.mcap) {  // (re)allocate the per-component ready words
        cudaFree(h->ws.mflags);
        cudaFree(h->ws.mrec);
        h->ws.mflags = nullptr;
        h->ws.mrec = nullptr;
        if ((!h->ws.mst && cudaMalloc(&h->ws.mst, sizeof(SolveState)) != cudaSuccess) ||
            cudaMalloc(&h->ws.mflags, 4 * words) != cudaSuccess || cudaMalloc(&h->ws.mrec, 16 * words) != cudaSuccess) {
            (void)cudaGetLastError();
            h->ws.mcap = 0;
            return SPTRSV_ERR_ALLOC;
        }
        h->ws.mcap = nrhs;
        h->mlaunch_key = -1;
    }
    int g = 1;
    while (g < nrhs) g *= 2;
    const int rows_per_cta = 256 / g;
    const unsigned grid = (unsigned)((h->n + rows_per_cta - 1) / rows_per_cta);
    const long long key = ((long long)grid << 8) | ((long long)nrhs << 1) | h->proto;
    if (key != h->mlaunch_key || reset_due(h->msince_reset, grid)) {
        CK(cudaMemsetAsync(h->ws.mflags, 0, 4 * words, s));
        CK(cudaMemsetAsync(h->ws.mrec, 0, 16 * words, s));
        h->mgen = (h->mgen + 1) & 0xFFFFFFu;
        const int rc = init_state(h->ws.mst, h->mgen, s);
        if (rc) return rc;
        h->mlaunch_key = key;
        h->msince_reset = 0;
    }
    SolveParams p = {};
    p.rowptr = h->rowptr;
    p.colidx = h->colidx;
    p.val = h->val;
    p.flags = h->ws.mflags;
    p.rec = h->ws.mrec;
    p.st = h->ws.mst;
    p.nnz = h->nnz;
    p.n = h->n;
    p.n_tasks = h->n_tasks;
    p.epoch0 = 1;
    p.gen = h->mgen;
    p.grid = grid;
    p.backoff_min = h->backoff_min;
    p.backoff_max = h->backoff_max;
    p.spin_limit = h->spin_limit;
    MultiParams m;
    m.B = B;
    m.X = X;
    m.ldb = ldb;
    m.ldx = ldx;
    m.nrhs = nrhs;
    m.g = g;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    cfg.numAttrs = 0;
    const cudaError_t e = h->proto ? cudaLaunchKernelEx(&cfg, k_solve_multi<PROTO_FUSED>, p, m)
                                   : cudaLaunchKernelEx(&cfg, k_solve_multi<PROTO_FLAGS>, p, m);
    if (e != cudaSuccess) {
        (void)cudaGetLastError();
        return SPTRSV_ERR_CUDA;
    }
    h->solves++;
    h->msince_reset++;
    return SPTRSV_OK;
}

int sptrsv_solve_host(sptrsv_handle_t h, const double *b_host, double *x_host, sptrsv_stream_t stream) {
    if (!h) return SPTRSV_ERR_INVALID_ARG;
    if (h->n == 0) return SPTRSV_OK;
    if (!b_host || !x_host) return SPTRSV_ERR_INVALID_ARG;
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess || cur != h->device) {
        (void)cudaGetLastError();
        return SPTRSV_ERR_INVALID_ARG;
    }
    Launch L0;
    const int rc0 = plan_launch(h, &L0);
    if (rc0) return rc0;
    const size_t bytes = sizeof(double) * (size_t)h->n;
    if (!h->ws.b_stage) {
        if (cudaMalloc(&h->ws.b_stage, bytes) != cudaSuccess) {
            (void)cudaGetLastError();
            return SPTRSV_ERR_ALLOC;
        }
    }
    if (!h->ws.x_stage) {
        if (cudaMalloc(&h->ws.x_stage, bytes) != cudaSuccess) {
            (void)cudaGetLastError();
            return SPTRSV_ERR_ALLOC;
        }
    }
    cudaStream_t s = (cudaStream_t)stream;
    // Pinned host buffers and the LEAN / CHAIN / HYBRID engines: b is copied in by DMA in ~4 chunks on a second
    // stream and each CTA of the solve waits only for the chunk holding its own rows, so the
    // host->device copy overlaps the solve; every LEAN CTA / CHAIN warp writes its finished rows of
    // x to host memory as one contiguous block (UVA mapping), so the device->host transfer overlaps
    // it too (HYBRID copies x back after the solve).  x still lands in device memory (the FLAGS
    // protocol reads it back; FUSED consumers read records).
    // c2, tools/e2e_probe.py: 270 us per step, against 357 us staged both ways and 330 us with
    // only the x side overlapped; reading b in-kernel over PCIe instead measured 469 us.
    cudaPointerAttributes ab, ax;
    const bool pinned = cudaPointerGetAttributes(&ab, b_host) == cudaSuccess &&
                        cudaPointerGetAttributes(&ax, x_host) == cudaSuccess && ab.type == cudaMemoryTypeHost &&
                        ax.type == cudaMemoryTypeHost && ab.devicePointer && ax.devicePointer;
    (void)cudaGetLastError();
    int io = h->host_io & 3;  // bit 0: b in chunks overlapped with the solve, bit 1: x written per CTA
    // b chunk = 2^sh rows: the option's bits 8.., else about four chunks (each copy + flag write costs
    // a few us of DMA setup; measured on c2: 2^15-row chunks 549 us, 2^16 394, 2^18 270, 2^20 324)
    int sh = h->host_io >> 8;
    if (!sh) {
        sh = kBChunkShift;
        while (sh < 24 && ((long long)4 << sh) < (long long)h->n) ++sh;
    }
    if ((io & 1) && !write_value32()) io &= ~1;
    // engines that take the chunked b (wait_b_chunks) and, for LEAN / CHAIN, write x per CTA / warp
    const int eng = L0.engine;
    const bool gated = eng == ENG_LEAN || eng == ENG_LEANP || eng == ENG_CHAIN || eng == ENG_HYBRID;
    if (pinned && io && eng == ENG_SMALL) {
        // SMALL: the one CTA reads b straight from the mapped pinned buffer (one coalesced pass over
        // PCIe, no copy launch) and writes x to both x_stage and the mapped pinned x
        int rc = solve_impl(h, (const double *)ab.devicePointer, h->ws.x_stage, (double *)ax.devicePointer, stream);
        if (rc) return rc;
        if (spin_sync(s, h->ws.ev_done)) return SPTRSV_ERR_CUDA;
        return SPTRSV_OK;
    }
    if (!(eng == ENG_LEAN || eng == ENG_LEANP || eng == ENG_CHAIN)) io &= ~2;
    if (pinned && io && gated) {
        const uint32_t *bflag = nullptr;
        uint32_t seq = 0;
        if (io & 1) {
            // b in chunks of 2^16 rows on a second stream; after each chunk a stream memory op sets
            // its flag to this call's sequence number, and a CTA of the solve waits for the flags
            // of its own rows only -- the copy and the solve overlap, chunk by chunk
            const int nch = (int)((h->n + (1 << sh) - 1) >> sh);
            Workspace &w = h->ws;
            if (w.bflag_n < nch) {
                cudaFree(w.bflag);
                w.bflag = nullptr;
                w.bflag_n = 0;
                if (cudaMalloc(&w.bflag, sizeof(uint32_t) * nch) != cudaSuccess) {
                    (void)cudaGetLastError();
                    return SPTRSV_ERR_ALLOC;
                }
                CK(cudaMemset(w.bflag, 0, sizeof(uint32_t) * nch));
                w.bflag_n = nch;
                h->host_seq = 0;
            }
            if (!w.s2) CK(cudaStreamCreateWithFlags(&w.s2, cudaStreamNonBlocking));
            if (!w.ev_a) CK(cudaEventCreateWithFlags(&w.ev_a, cudaEventDisableTiming));
            if (!w.ev_b) CK(cudaEventCreateWithFlags(&w.ev_b, cudaEventDisableTiming));
            seq = ++h->host_seq;
            if (seq == 0) seq = ++h->host_seq;  // 0 is the reset value (wrap-safe compare in the kernel)
            CK(cudaEventRecord(w.ev_a, s));  // the copies start after the stream's earlier work
            CK(cudaStreamWaitEvent(w.s2, w.ev_a, 0));
            for (int c = 0; c < nch; ++c) {
                const size_t r0 = (size_t)c << sh;
                const size_t rows = std::min((size_t)h->n - r0, (size_t)1 << sh);
                CK(cudaMemcpyAsync(w.b_stage + r0, b_host + r0, rows * sizeof(double), cudaMemcpyHostToDevice,
                                   w.s2));
                if (write_value32()(w.s2, (unsigned long long)(uintptr_t)(w.bflag + c), seq, 0) != 0)
                    return SPTRSV_ERR_CUDA;
            }
            bflag = w.bflag;
        } else {
            CK(cudaMemcpyAsync(h->ws.b_stage, b_host, bytes, cudaMemcpyHostToDevice, s));
        }
        int rc = solve_impl(h, h->ws.b_stage, h->ws.x_stage, (io & 2) ? (double *)ax.devicePointer : nullptr, stream,
                            bflag, seq, sh, /*host_state=*/true);
        if (rc) return rc;
        if (io & 1) {  // the stream also orders after the copies (they finish before the solve does)
            CK(cudaEventRecord(h->ws.ev_b, h->ws.s2));
            CK(cudaStreamWaitEvent(s, h->ws.ev_b, 0));
        }
        if (!(io & 2)) CK(cudaMemcpyAsync(x_host, h->ws.x_stage, bytes, cudaMemcpyDeviceToHost, s));
        if (spin_sync(s, h->ws.ev_done)) return SPTRSV_ERR_CUDA;
        return SPTRSV_OK;
    }
    CK(cudaMemcpyAsync(h->ws.b_stage, b_host, bytes, cudaMemcpyHostToDevice, s));
    int rc = sptrsv_solve(h, h->ws.b_stage, h->ws.x_stage, stream);
    if (rc) return rc;
    CK(cudaMemcpyAsync(x_host, h->ws.x_stage, bytes, cudaMemcpyDeviceToHost, s));
    if (spin_sync(s, h->ws.ev_done)) return SPTRSV_ERR_CUDA;
    return SPTRSV_OK;
}

int sptrsv_destroy(sptrsv_handle_t h) {
    if (!h) return SPTRSV_OK;
    DeviceGuard g(h->device);
    cudaDeviceSynchronize();
    if (h->l2_user) {
        // demote this handle's persisting lines only (a context-wide reset would demote every
        // other handle's window too): discard the window's L2 lines -- the records are dead
        void *wbase = h->proto == PROTO_FLAGS ? (void *)h->ws.flags : (void *)h->ws.rec;
        const size_t wbytes = (h->proto == PROTO_FLAGS ? sizeof(uint32_t) : 16) * (size_t)h->n;
        if (wbase) {
            k_l2_discard<<<(unsigned)std::min<size_t>((wbytes / 128 + 255) / 256, 4096), 256>>>(
                (char *)wbase, wbytes);
            cudaDeviceSynchronize();
        }
        l2_limit_release(h);
    }
    (void)cudaGetLastError();
    free_ws(h->ws);
    cudaFree(h->own_rowptr);
    cudaFree(h->own_colidx);
    cudaFree(h->own_val);
    delete h;
    return SPTRSV_OK;
}

int sptrsv_set_option(sptrsv_handle_t h, int key, int64_t value) {
    if (!h) return SPTRSV_ERR_INVALID_ARG;
    if (h->tri && key == SPTRSV_OPT_VARIANT && value != 0)
        return SPTRSV_ERR_INVALID_ARG;  // the paper's kernels are lower-only
    DeviceGuard g(h->device);
    switch (key) {
        case SPTRSV_OPT_MODE:
            if (value < 0 || value > 3) return SPTRSV_ERR_INVALID_ARG;
            h->mode = (int)value;
            return build_plan(h);
        case SPTRSV_OPT_WARP_THRESHOLD:
            if (value < 0 || value > (1 << 30)) return SPTRSV_ERR_INVALID_ARG;
            h->threshold = (int)value;
            h->threshold_user = true;
            return build_plan(h);
        case SPTRSV_OPT_CTA_THREADS:
            if (value != 0 && value != 32 && value != 64 && value != 128 && value != 256 && value != 512 && value != 1024)
                return SPTRSV_ERR_INVALID_ARG;
            h->cta_threads = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_BACKOFF_MIN_NS:
            if (value < 0 || value > 1000000) return SPTRSV_ERR_INVALID_ARG;
            h->backoff_min = (uint32_t)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_BACKOFF_MAX_NS:
            if (value < 0 || value > 1000000) return SPTRSV_ERR_INVALID_ARG;
            h->backoff_max = (uint32_t)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_SPIN_LIMIT:
            if (value < 0 || value > 0xFFFFFFFFll) return SPTRSV_ERR_INVALID_ARG;
            h->spin_limit = (uint32_t)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_L2_WINDOW:
            if (value != 0 && value != 1) return SPTRSV_ERR_INVALID_ARG;
            h->l2_window = (int)value;
            size_l2_window(h);
            return SPTRSV_OK;
        case SPTRSV_OPT_STAGE_SMEM:
            if (value != 0 && value != 1) return SPTRSV_ERR_INVALID_ARG;
            h->stage = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_PROTOCOL:
            if (value != PROTO_FLAGS && value != PROTO_FUSED) return SPTRSV_ERR_INVALID_ARG;
            h->proto = (int)value;  // both kinds of ready words live in the workspace; the next solve re-zeroes
            size_l2_window(h);
            return SPTRSV_OK;
        case SPTRSV_OPT_LOCAL:
            if (value != 0 && value != 1) return SPTRSV_ERR_INVALID_ARG;
            h->local = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_ENGINE:
            if (value != ENG_ONESHOT && value != ENG_LEAN && value != ENG_AUTO && value != ENG_HYBRID &&
                value != ENG_CHAIN && value != ENG_SMALL && value != ENG_LEANP && value != ENG_GRID)
                return SPTRSV_ERR_INVALID_ARG;
            if (value == ENG_SMALL && !small_fits(h)) return SPTRSV_ERR_INVALID_ARG;  // does not fit one CTA
            if (value == ENG_GRID && !grid_ok(h)) return SPTRSV_ERR_INVALID_ARG;    // not grid-shaped
            h->engine = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_ROWS_PER_LANE:
            if (value < 0 || value > 2) return SPTRSV_ERR_INVALID_ARG;
            h->rows_per_lane = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_VARIANT:
            if (value != 0 && value != 3 && value != 4 && value != 5) return SPTRSV_ERR_INVALID_ARG;
            h->variant = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_LEAN_OCCUPANCY:
            if (value < 5 || value > 8) return SPTRSV_ERR_INVALID_ARG;
            h->lean_minb = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_POLL_GAP_NS:
            if (value < 0 || value > 1000000) return SPTRSV_ERR_INVALID_ARG;
            h->poll_gap = (uint32_t)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_POLL_ONE:
            if (value != 0 && value != 1) return SPTRSV_ERR_INVALID_ARG;
            h->poll_one = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_HOST_IO:  // bits 0-1 mode, bits 8.. log2 of the b chunk in rows (0 = 16)
            if ((value & ~0xFF03ll) || ((value >> 8) && ((value >> 8) < 8 || (value >> 8) > 24)))
                return SPTRSV_ERR_INVALID_ARG;
            h->host_io = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_CHAIN_DIV:
            if (value < 0 || value > 2) return SPTRSV_ERR_INVALID_ARG;
            h->chain_div = (int)value;
            return SPTRSV_OK;
        case SPTRSV_OPT_SUBWARP:
            if (value < 0 || value > 64) return SPTRSV_ERR_INVALID_ARG;
            h->subwarp_epl = (int)value;
            return build_plan(h);
        case SPTRSV_OPT_WARP_SPLIT_LAST:
            if (value < 0 || value > 2) return SPTRSV_ERR_INVALID_ARG;
            h->split_last = (int)value;
            return SPTRSV_OK;
        default:
            return SPTRSV_ERR_INVALID_ARG;
    }
}

int sptrsv_get_option(sptrsv_handle_t h, int key, int64_t *value) {
    if (!h || !value) return SPTRSV_ERR_INVALID_ARG;
    switch (key) {
        case SPTRSV_OPT_MODE: *value = h->mode; return SPTRSV_OK;
        case SPTRSV_OPT_WARP_THRESHOLD: *value = h->threshold; return SPTRSV_OK;
        case SPTRSV_OPT_CTA_THREADS: *value = h->cta_threads; return SPTRSV_OK;
        case SPTRSV_OPT_BACKOFF_MIN_NS: *value = h->backoff_min; return SPTRSV_OK;
        case SPTRSV_OPT_BACKOFF_MAX_NS: *value = h->backoff_max; return SPTRSV_OK;
        case SPTRSV_OPT_SPIN_LIMIT: *value = h->spin_limit; return SPTRSV_OK;
        case SPTRSV_OPT_L2_WINDOW: *value = h->l2_window; return SPTRSV_OK;
        case SPTRSV_OPT_STAGE_SMEM: *value = h->stage; return SPTRSV_OK;
        case SPTRSV_OPT_PROTOCOL: *value = h->proto; return SPTRSV_OK;
        case SPTRSV_OPT_LOCAL: *value = h->local; return SPTRSV_OK;
        case SPTRSV_OPT_ENGINE: *value = h->engine; return SPTRSV_OK;
        case SPTRSV_OPT_ROWS_PER_LANE: *value = h->rows_per_lane; return SPTRSV_OK;
        case SPTRSV_OPT_VARIANT: *value = h->variant; return SPTRSV_OK;
        case SPTRSV_OPT_LEAN_OCCUPANCY: *value = h->lean_minb; return SPTRSV_OK;
        case SPTRSV_OPT_POLL_GAP_NS: *value = h->poll_gap; return SPTRSV_OK;
        case SPTRSV_OPT_POLL_ONE: *value = h->poll_one; return SPTRSV_OK;
        case SPTRSV_OPT_WARP_SPLIT_LAST: *value = h->split_last; return SPTRSV_OK;
        case SPTRSV_OPT_HOST_IO: *value = h->host_io; return SPTRSV_OK;
        case SPTRSV_OPT_CHAIN_DIV: *value = h->chain_div; return SPTRSV_OK;
        case SPTRSV_OPT_SUBWARP: *value = h->subwarp_epl >= 0 ? h->subwarp_epl : h->epl_eff; return SPTRSV_OK;
        default: return SPTRSV_ERR_INVALID_ARG;
    }
}

int sptrsv_get_info(sptrsv_handle_t h, sptrsv_info *out) {
    if (!h || !out) return SPTRSV_ERR_INVALID_ARG;
    out->n = h->n;
    out->nnz = h->nnz;
    out->n_thread_groups = h->n_thread_groups;
    out->n_warp_rows = h->n_warp_rows;
    out->n_sub_tasks = h->n_sub_tasks;
    out->n_tasks = h->n_tasks;
    out->max_row_nnz = h->max_row;
    out->device = h->device;
    out->analyse_ms = h->analyse_ms;
    out->solves = h->solves;
    out->near_deps = h->near_deps;
    out->warp_deps = h->warp_deps;
    out->prev_deps = h->prev_deps;
    out->near_rows = h->near_rows;
    Launch L;
    const int rc = plan_launch(h, &L);
    if (rc) return rc;
    out->engine = L.engine;
    out->cta_threads = L.cta;
    out->rows_per_lane = L.K;
    return SPTRSV_OK;
}

int sptrsv_get_indegree(sptrsv_handle_t h, int32_t *out_dev, sptrsv_stream_t stream) {
    if (!h || (!out_dev && h->n > 0)) return SPTRSV_ERR_INVALID_ARG;
    if (h->n == 0) return SPTRSV_OK;
    DeviceGuard g(h->device);
    CK(cudaMemcpyAsync(out_dev, h->ws.indeg, sizeof(int32_t) * (size_t)h->n, cudaMemcpyDeviceToDevice,
                       (cudaStream_t)stream));
    return SPTRSV_OK;
}

int sptrsv_levels(sptrsv_handle_t h, int32_t *level_dev, int32_t *counts_dev, int32_t *nlevels_host,
                  sptrsv_stream_t stream) {
    if (!h || !nlevels_host || h->tri) return SPTRSV_ERR_INVALID_ARG;
    *nlevels_host = 0;
    if (h->n == 0) return SPTRSV_OK;
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    const size_t n = (size_t)h->n;
    if (!h->ws.lvl) {
        if (cudaMalloc(&h->ws.lvl, sizeof(uint32_t) * (n + 1)) != cudaSuccess) {
            (void)cudaGetLastError();
            return SPTRSV_ERR_ALLOC;
        }
    }
    int32_t *d_nlev = reinterpret_cast<int32_t *>(h->ws.lvl + n);
    CK(cudaMemsetAsync(h->ws.lvl, 0, sizeof(uint32_t) * (n + 1), s));
    CK(cudaMemsetAsync(&h->ws.st->lticket.v, 0, sizeof(uint32_t), s));
    if (counts_dev) CK(cudaMemsetAsync(counts_dev, 0, sizeof(int32_t) * n, s));
    const int groups = (h->n + 31) / 32;
    k_levels<<<(groups + 7) / 8, 256, 0, s>>>(h->rowptr, h->colidx, h->ws.lvl, h->ws.st, h->n);
    CK(cudaGetLastError());
    k_level_finish<<<(h->n + 255) / 256, 256, 0, s>>>(h->ws.lvl, level_dev, counts_dev, d_nlev, h->n);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(nlevels_host, d_nlev, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    return SPTRSV_OK;
}

int sptrsv_set_trace(sptrsv_handle_t h, uint64_t *trace_dev) {
    if (!h) return SPTRSV_ERR_INVALID_ARG;
    h->trace = reinterpret_cast<unsigned long long *>(trace_dev);
    return SPTRSV_OK;
}

int sptrsv_check(sptrsv_handle_t h, sptrsv_stream_t stream) {
    if (!h) return SPTRSV_ERR_INVALID_ARG;
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    CK(cudaStreamSynchronize(s));
    uint32_t err = 0, merr = 0;
    CK(cudaMemcpy(&err, &h->ws.st->error.v, sizeof(uint32_t), cudaMemcpyDeviceToHost));
    if (h->ws.mst) {
        CK(cudaMemcpy(&merr, &h->ws.mst->error.v, sizeof(uint32_t), cudaMemcpyDeviceToHost));
        if (merr) {
            CK(cudaMemset(h->ws.mst, 0, sizeof(SolveState)));
            h->mlaunch_key = -1;
        }
    }
    if (h->ws.hst && !merr) {  // the host-path state of a LEANP handle (its own epoch sequence)
        CK(cudaMemcpy(&merr, &h->ws.hst->error.v, sizeof(uint32_t), cudaMemcpyDeviceToHost));
        if (merr) {
            CK(cudaMemset(h->ws.hst, 0, sizeof(SolveState)));
            h->hlaunch_key = -1;
        }
    }
    if (err) {
        CK(cudaMemset(&h->ws.st->error.v, 0, sizeof(uint32_t)));
        CK(cudaMemset(&h->ws.st->abort.v, 0, sizeof(uint32_t)));
        h->launch_key = -1;  // flags of the aborted solve are partial: re-zero before the next one
    }
    const uint32_t e = err ? err : merr;
    if (e == kErrStale) return SPTRSV_ERR_STALE_LAUNCH;
    if (e == kErrInexact) {  // a CHAIN quotient failed its proof: prove every quotient in-loop from now on
        h->chain_div = 1;
        return SPTRSV_ERR_INEXACT;
    }
    return e ? SPTRSV_ERR_TIMEOUT : SPTRSV_OK;
}

int sptrsv_hop_scan(int32_t iters, int32_t protocol, int32_t capacity, int32_t *sm_a_out, int32_t *sm_b_out,
                    double *ns_out, int32_t *count) {
    constexpr int kHopAddrs = 8;
    if (iters <= 0 || (protocol != 0 && protocol != 1) || capacity < 0 || !count || !sm_a_out ||
        (capacity > 0 && (!sm_b_out || !ns_out)))
        return SPTRSV_ERR_INVALID_ARG;
    *count = 0;
    int dev = 0, nsm = 0, smem_sm = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev) ||
        cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev)) {
        (void)cudaGetLastError();
        return SPTRSV_ERR_CUDA;
    }
    const int smem = smem_sm / 2 + 1024;  // > half an SM: one CTA per SM
    if (cudaFuncSetAttribute(k_smids, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess ||
        cudaFuncSetAttribute(k_pingpong_sm, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) {
        (void)cudaGetLastError();
        return SPTRSV_ERR_CUDA;
    }
    unsigned long long *rec = nullptr, *ns = nullptr;
    uint32_t *flags = nullptr;
    double *xs = nullptr, *sink = nullptr;
    int32_t *ids = nullptr;
    int rc = SPTRSV_OK;
    do {
        if (cudaMalloc(&rec, 4096 * kHopAddrs) != cudaSuccess || cudaMalloc(&flags, 4096 * kHopAddrs) != cudaSuccess ||
            cudaMalloc(&xs, 512) != cudaSuccess || cudaMalloc(&sink, 16) != cudaSuccess ||
            cudaMalloc(&ns, 16) != cudaSuccess || cudaMalloc(&ids, sizeof(int32_t) * nsm) != cudaSuccess) {
            rc = SPTRSV_ERR_ALLOC;
            break;
        }
        std::vector<int32_t> h_ids(nsm);
        k_smids<<<nsm, 32, smem>>>(ids);
        if (cudaGetLastError() != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess ||
            cudaMemcpy(h_ids.data(), ids, sizeof(int32_t) * nsm, cudaMemcpyDeviceToHost) != cudaSuccess) {
            rc = SPTRSV_ERR_CUDA;
            break;
        }
        std::sort(h_ids.begin(), h_ids.end());
        h_ids.erase(std::unique(h_ids.begin(), h_ids.end()), h_ids.end());
        const int a = h_ids[0];
        *sm_a_out = a;
        for (size_t k = 1; k < h_ids.size() && *count < capacity; ++k) {
            // the ready words' L2 slice (and its die) follows the address: every pair is measured at
            // kAddrs addresses 4 KB apart and keeps the fastest -- the hop of the best placement
            double best = 1e30;
            for (int ad = 0; ad < kHopAddrs && rc == SPTRSV_OK; ++ad) {
                unsigned long long *r = rec + (size_t)ad * 512;
                uint32_t *f = flags + (size_t)ad * 1024;
                if (cudaMemset(r, 0, 512) != cudaSuccess || cudaMemset(f, 0, 512) != cudaSuccess) {
                    rc = SPTRSV_ERR_CUDA;
                    break;
                }
                k_pingpong_sm<<<nsm, 32, smem>>>(r, f, xs, iters, protocol, a, h_ids[k], ns, sink);
                unsigned long long t = 0;
                if (cudaGetLastError() != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess ||
                    cudaMemcpy(&t, ns, 8, cudaMemcpyDeviceToHost) != cudaSuccess) {
                    rc = SPTRSV_ERR_CUDA;
                    break;
                }
                best = std::min(best, (double)t / (2.0 * iters));
            }
            if (rc) break;
            sm_b_out[*count] = h_ids[k];
            ns_out[*count] = best;
            ++*count;
        }
    } while (0);
    (void)cudaGetLastError();
    cudaFree(rec);
    cudaFree(flags);
    cudaFree(xs);
    cudaFree(sink);
    cudaFree(ns);
    cudaFree(ids);
    return rc;
}

int sptrsv_flag_latency(int32_t iters, int32_t protocol, double *ns_per_hop, double *sm_mhz) {
    if (iters <= 0 || protocol < 0 || protocol > 7 || !ns_per_hop) return SPTRSV_ERR_INVALID_ARG;
    uint32_t *flags = nullptr;
    double *xs = nullptr, *sink = nullptr;
    unsigned long long *ns = nullptr;
    int rc = SPTRSV_OK;
    do {
        if (cudaMalloc(&flags, 256) != cudaSuccess || cudaMalloc(&xs, 256) != cudaSuccess ||
            cudaMalloc(&sink, 16) != cudaSuccess || cudaMalloc(&ns, 16) != cudaSuccess) {
            rc = SPTRSV_ERR_ALLOC;
            break;
        }
        if (cudaMemset(flags, 0, 256) != cudaSuccess || cudaMemset(xs, 0, 256) != cudaSuccess) {
            rc = SPTRSV_ERR_CUDA;
            break;
        }
        k_pingpong<<<2, 32>>>(flags, xs, iters, protocol, ns, sink);
        unsigned long long t[2] = {0, 0};
        if (cudaGetLastError() != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess ||
            cudaMemcpy(t, ns, 16, cudaMemcpyDeviceToHost) != cudaSuccess) {
            rc = SPTRSV_ERR_CUDA;
            break;
        }
        // hops: 2 per iteration for the ping-pong protocols, 1 per iteration for the probes
        *ns_per_hop = (double)t[0] / ((protocol >= 3 ? 1.0 : 2.0) * iters);
        if (sm_mhz) *sm_mhz = t[0] ? (double)t[1] / (double)t[0] * 1e3 : 0.0;
    } while (0);
    (void)cudaGetLastError();
    cudaFree(flags);
    cudaFree(xs);
    cudaFree(sink);
    cudaFree(ns);
    return rc;
}

}  // extern "C"
