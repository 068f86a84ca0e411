/*
 * sptrsv.h -- C ABI of the B200-native CapelliniSpTRSV hot path.
 *
 * Operation (sec.1; Alg.1): solve L x = b for x,
 * L an n x n sparse LOWER-triangular matrix in CSR form, b and x dense fp64:
 *     x_i = (b_i - sum_{j<i, L_ij stored} L_ij * x_j) / L_ii ,  i = 0..n-1.
 * Method (Alg.5 "Writing-First CapelliniSpTRSV"): no level
 * preprocessing; one GPU thread per component x_i in original row order, which
 * busy-waits on per-component ready flags of its dependencies, accumulates the
 * partial sum, then publishes x_i.  Rows whose 32-row group has a high mean
 * nnz/row are solved one WARP per row instead (the thread/warp hybrid the paper
 * proposes in sec.4.4; warp kernel = Alg.3).
 *
 * All functions are host functions and thread-compatible (one handle must not
 * be used from two host threads at once).  Pointers documented "device" must
 * be device pointers valid on the CURRENT CUDA device (e.g. a torch tensor's
 * data_ptr()); "host" pointers are ordinary host memory.  Streams are passed as
 * sptrsv_stream_t, which is a cudaStream_t (NULL = the legacy default stream).
 * No torch or CUDA types appear in this header.
 *
 * Return value: every function returns SPTRSV_OK (0) or a negative
 * sptrsv_status.  sptrsv_strerror() maps a status to a static string.
 */
#ifndef SPTRSV_H_
#define SPTRSV_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SPTRSV_ABI_VERSION 4

typedef struct sptrsv_handle_s *sptrsv_handle_t;
typedef void *sptrsv_stream_t; /* cudaStream_t */

typedef enum sptrsv_status {
    SPTRSV_OK = 0,
    SPTRSV_ERR_INVALID_ARG = -1,  /* null pointer, n < 0, bad option value ...             */
    SPTRSV_ERR_NOT_LOWER = -2,    /* a stored column j > i                                  */
    SPTRSV_ERR_MISSING_DIAG = -3, /* empty row, or the last stored column of row i != i     */
    SPTRSV_ERR_ZERO_DIAG = -4,    /* L_ii == 0                                              */
    SPTRSV_ERR_UNSORTED = -5,     /* columns of a row not strictly increasing (dup/unsorted) */
    SPTRSV_ERR_BAD_ROWPTR = -6,   /* rowptr[0] != 0, decreasing, or entry beyond rowptr[n]  */
    SPTRSV_ERR_BAD_COL = -7,      /* a column index < 0                                     */
    SPTRSV_ERR_TOO_LARGE = -8,    /* n > 2^31 - 2 (int32 CSR)                  */
    SPTRSV_ERR_CUDA = -9,         /* a CUDA runtime call failed (launch, copy, ...)         */
    SPTRSV_ERR_ALLOC = -10,       /* device / pinned allocation failed                      */
    SPTRSV_ERR_TIMEOUT = -11,     /* watchdog: a solve spun past SPTRSV_OPT_SPIN_LIMIT      */
    SPTRSV_ERR_INEXACT = -13,     /* a CHAIN solve found a quotient that failed its exactness
                                     proof (never observed): the solve
                                     was aborted and the handle switched to in-loop proofs
                                     (SPTRSV_OPT_CHAIN_DIV = 1); re-solve                   */
    SPTRSV_ERR_STALE_LAUNCH = -12 /* a solve captured in a CUDA graph was replayed after the
                                     handle's launch configuration changed (an option
                                     change or a watchdog reset re-zeroes the ready words
                                     under a new generation): the stale launch did not
                                     solve; re-capture the graph                           */
} sptrsv_status;

/* Options (sptrsv_set_option / sptrsv_get_option).  None changes the result
 * beyond fp64 summation order (warp mode sums lane-strided partials). */
typedef enum sptrsv_option {
    SPTRSV_OPT_MODE = 1,           /* 0 AUTO (default), 1 THREAD (every row thread-level,
                                      Alg.5), 2 WARP (every row warp-level, Alg.3), 3 SUB-WARP
                                      (every 32-row group at the sub-warp width its mean
                                      nnz/row gives, see SPTRSV_OPT_SUBWARP).
                                      Setting it re-plans (synchronous).                    */
    SPTRSV_OPT_WARP_THRESHOLD = 2, /* AUTO: a 32-row group goes warp-level when its mean
                                      nnz/row exceeds this.  Default: derived at analyse from
                                      the median distance to each row's nearest dependency
                                      (< 64 rows: never; 64-1023: 2; 1024-8191: 6; wider: 20;
                                      n <= 1024: never; sec.4.4, DESIGN G10).  Setting it
                                      overrides that and re-plans (synchronous).            */
    SPTRSV_OPT_CTA_THREADS = 3,    /* threads per CTA, or 0 (default) = the engine's measured
                                      best: 32, 64, 128, 256, 512 or 1024.  ONE-SHOT: 64..1024;
                                      LEAN (lower): 128, 256, 512; CHAIN: 64, 128, 256;
                                      HYBRID: 64, 256; SMALL: any (capped at n rounded up to
                                      a warp); other values / engines: default             */
    SPTRSV_OPT_BACKOFF_MIN_NS = 4, /* __nanosleep after a pass where no lane progressed     */
    SPTRSV_OPT_BACKOFF_MAX_NS = 5, /* exponential backoff cap                               */
    SPTRSV_OPT_SPIN_LIMIT = 6,     /* watchdog: idle passes per warp before TIMEOUT (0=off) */
    SPTRSV_OPT_L2_WINDOW = 7,      /* 1 (default): a persisting cudaAccessPolicyWindow over
                                      the ready words (FLAGS: flags, FUSED: records); the
                                      device's persisting L2 set-aside is grown to the window
                                      (up to persistingL2CacheMaxSize) at the first solve;
                                      ready words larger than that run without a window.
                                      0: no window                                         */
    SPTRSV_OPT_STAGE_SMEM = 8,     /* 1 (default): thread-level warps stage their CSR slice
                                      in shared memory with coalesced loads                 */
    SPTRSV_OPT_PROTOCOL = 9,       /* cross-CTA ready protocol: 0 FLAGS = uint32 epoch flags,
                                      st.release.gpu / ld.acquire.gpu (Alg.5 l.15-16 + DESIGN
                                      G6); 1 FUSED (default) = 16-byte record per component,
                                      each 8-byte half = epoch<<32 | half of x_i, no fences
                                                                     */
    SPTRSV_OPT_LOCAL = 10,         /* 1 (default): dependencies produced inside the same CTA
                                      are read from a shared-memory copy of x               */
    SPTRSV_OPT_ENGINE = 11,        /* 5 (default) AUTO, from analyse's statistics (DESIGN.md
                                      section 6): SMALL for systems of <= 4096 rows with
                                      near dependencies that are not pure chains and whose
                                      CSR, b and x fit one CTA's shared memory (24 B per
                                      row + 12 B per entry <= 226 KB);
                                      else GRID for grid-shaped lower factors (see 10);
                                      else HYBRID for plans with warp-level rows; for
                                      all-thread-level plans LEANP when < 1/4 of the rows
                                      wait on a row < 256 away, CHAIN for long runs of
                                      previous-row dependencies (>= 1/4 of the dependencies,
                                      mean run >= 2048 rows, runs starting on 64-row
                                      boundaries), else ONE-SHOT.
                                      Forced engines:
                                      0 ONE-SHOT (lower): one CTA per row range, ticketed,
                                      smem-staged CSR slices, in-CTA x copy in smem;
                                      3 LEAN: minimal-latency kernel, one row per lane, no
                                      staging, speculative rows;
                                      6 HYBRID: one task per warp -- a warp-level row (Alg.3)
                                      or a 32-row thread group (LEAN's per-lane loop);
                                      7 CHAIN: in-warp dependency chains resolved in
                                      registers / shared memory, external ones by polling;
                                      8 SMALL: one CTA, the whole system in shared memory
                                      (any plan, any triangular form; INVALID_ARG when it
                                      does not fit; CTA_THREADS: 32..1024, multiple of 32);
                                      9 LEANP: LEAN's row loop in persistent warps (a
                                      cooperative launch of what fits on the device, static
                                      round-robin blocks) with the next chunks' loads in
                                      flight during the current chunk's waits;
                                      10 GRID: wavefront bands for stencil-shaped factors
                                      (any triangular form, in logical rows: rows depending
                                      only on their west r-1 / north r-m neighbours and at
                                      most one far row in an earlier band / step, m found by
                                      analyse; upper handles need n % m == 0): lane l of a band's warp owns grid column
                                      32k+l, north operands stay in registers, west ones
                                      move by shuffle, one protocol hop per 32 columns.
                                      AUTO takes it (FUSED protocol) for 2D grids (<= 1/8 far
                                      entries) with m >= 32 columns and >= 32 lines; forcing
                                      it on a matrix that is not grid-shaped returns
                                      INVALID_ARG.
                                      LEAN, LEANP and CHAIN need an all-thread-level plan; a
                                      plan with warp-level rows runs HYBRID (ONE-SHOT if
                                      forced on a lower handle).  sptrsv_info.engine reports
                                      the engine that runs.  Other values: INVALID_ARG      */
    /* 12, 13, 14: retired (the PIPE ablation engine left the library in round 2)       */
    SPTRSV_OPT_ROWS_PER_LANE = 15, /* CHAIN: K = 1 or 2 (0 = default 2) rows per lane       */
    SPTRSV_OPT_LEAN_OCCUPANCY = 17,/* LEAN engine register budget: 5..8 (default 5)
                                      resident 256-thread CTAs per SM                       */
    /* 18: retired (the L2 bulk prefetch of LEAN measured no gain and left in round 2)   */
    SPTRSV_OPT_POLL_GAP_NS = 19,   /* LEAN: __nanosleep after a pass that progressed but left
                                      lanes waiting (0 = default, none)                    */
    SPTRSV_OPT_POLL_ONE = 20,      /* LEAN: 1 = poll one dependency per lane per pass
                                      (default 0: the next two, DESIGN G21)                 */
    SPTRSV_OPT_SUBWARP = 24,       /* sub-warp rows (the thread-vs-warp granularity
                                      of sec.4.4): a 32-row group that AUTO
                                      takes beyond thread level runs W lanes per row, W the
                                      smallest power of two in [2, 32] with W * value >= its
                                      mean off-diagonals per row (32 / W rows per warp task,
                                      segmented lane tree).  value = target off-diagonals per
                                      lane, 1..64; 0 = one warp per row (Alg.3) for every
                                      such group.  Default: AUTO picks it (and the threshold)
                                      from the median nearest-dependency distance (DESIGN.md
                                      section 6); AUTO caps W at 16.  Setting it re-plans
                                      (synchronous).                                        */
    SPTRSV_OPT_CHAIN_DIV = 25,     /* CHAIN's division proof (Diag::exact, DESIGN.md section
                                      6): 0 (default) = the chain runs the Markstein candidate
                                      and proves each run's quotients right after it, all
                                      lanes in parallel (a failure aborts the solve with
                                      SPTRSV_ERR_INEXACT); 1 = prove every quotient before the
                                      chain uses it (+~25 cycles per chain step); 2 = test
                                      hook: every post-run proof fails.  SMALL always proves
                                      after its sweep and, on a failure, re-runs the sweep
                                      with the verified division (no error; 2 forces it)    */
    SPTRSV_OPT_HOST_IO = 23,       /* sptrsv_solve_host with pinned buffers on LEAN: bit 0 =
                                      b copied in chunks on a second stream, each CTA waiting
                                      for its own chunk only (needs cuStreamWriteValue32);
                                      bit 1 = each CTA writes its rows of x to host memory;
                                      a cleared bit uses one cudaMemcpyAsync before / after
                                      the solve instead.  Bits 8..15: log2 of the chunk in
                                      rows (8..24; 0 = about four chunks).  Default 3      */
    SPTRSV_OPT_WARP_SPLIT_LAST = 22,/* warp-level rows: 2 (default) = the row's last
                                      off-diagonal (its nearest dependency) is added after
                                      the lane-strided tree by lane 0 alone, which polls it
                                      with at most 32 ns sleeps; 1 = the same with the
                                      handle's backoff; 0 = it is part of the tree.  Every
                                      order is fixed (deterministic)                       */
    /* 21: retired (CHAIN publishes every finalized row at once)                        */
    SPTRSV_OPT_VARIANT = 16        /* ablation: 0 (default) product path; 3, 4, 5
                                      = the paper's Alg.3 SyncFree (warp per row), Alg.4
                                      Two-Phase, Alg.5 Writing-First with their printed
                                      control flow (FLAGS protocol, solve_paper.cuh)        */
} sptrsv_option;

typedef struct sptrsv_info {
    int32_t n;
    int32_t n_thread_groups;  /* 32-row groups solved thread-level                       */
    int64_t nnz;              /* rowptr[n]                                                */
    int32_t n_warp_rows;      /* rows solved warp-level                                   */
    int32_t n_tasks;          /* warp tasks per solve = n_thread_groups + n_warp_rows +
                                 n_sub_tasks                                               */
    int32_t max_row_nnz;      /* longest row (incl. diagonal)                             */
    int32_t device;           /* CUDA ordinal the handle is bound to                      */
    float analyse_ms;         /* wall time of sptrsv_analyse_csr (Table 1 analogue)        */
    uint32_t solves;          /* solves enqueued through this handle                      */
    int64_t near_deps;        /* dependencies with i - j < 256 (analyse statistic)         */
    int64_t warp_deps;        /* dependencies inside the row's own 32-row group            */
    int32_t engine;           /* engine the next solve launches (0 ONE-SHOT, 3 LEAN,
                                 6 HYBRID, 7 CHAIN, 8 SMALL, 9 LEANP, 10 GRID; 33/34/35
                                 the paper's Alg.3/4/5)                                    */
    int32_t cta_threads;      /* CTA size the next solve uses (defaults resolved)          */
    int32_t rows_per_lane;    /* rows per lane the next solve uses (defaults resolved)     */
    int64_t prev_deps;        /* dependencies on the previous row in solve order (i - 1;
                                 i + 1 for upper handles): AUTO's CHAIN criterion           */
    int32_t n_sub_tasks;      /* warp tasks holding 32/W sub-warp rows (W = 2..16 lanes per row) */
    int32_t pad_;
    int64_t near_rows;        /* rows whose nearest dependency is < 256 rows away: AUTO's
                                 LEAN criterion (LEAN when < n/4)                          */
} sptrsv_info;

/*
 * sptrsv_analyse_csr -- O(nnz) setup; the paper's "MALLOC(get_value, m)"
 * (Alg.5 l.1) plus the nnz-per-row pass the hybrid needs
 * (sec.4.4).  No level analysis, no reordering, no format
 * conversion.
 *   n       number of rows/columns, 0 <= n <= 2^31 - 2.
 *   rowptr  device, int32[n+1]; rowptr[0] = 0, nondecreasing; nnz = rowptr[n].
 *   colidx  device, int32[nnz]; per row strictly increasing, all <= i, and the
 *           diagonal (column i) stored LAST (Alg.1 l.5).
 *   val     device, double[nnz]; val[rowptr[i+1]-1] = L_ii != 0.
 *   out     host; receives the new handle (NULL on error).
 * Ownership: rowptr/colidx/val are BORROWED -- the caller keeps them alive and
 * unmodified until sptrsv_destroy.  The handle owns its workspace (flags,
 * in-degrees, task list, solve state).
 * Synchronous: runs on the legacy default stream and blocks until done; the
 * caller must have completed any writes to the CSR arrays.  Malformed input
 * returns the error of the lowest offending row (codes above) -- it never
 * reaches the spin loop, where it could hang.  Binds the handle to the
 * current device.
 */
int sptrsv_analyse_csr(int32_t n, const int32_t *rowptr, const int32_t *colidx,
                       const double *val, sptrsv_handle_t *out);

/* Triangular-form flags of sptrsv_analyse_csr_ex. */
#define SPTRSV_TRI_UPPER 1     /* U x = b: entries j >= i, diagonal stored FIRST in each row */
#define SPTRSV_TRI_UNIT_DIAG 2 /* diagonal implicitly 1 and NOT stored; rows may be empty    */

/*
 * sptrsv_analyse_csr_ex -- sptrsv_analyse_csr for the other triangular forms
 * (the paper solves L x = b only, Alg.1 :82-92;
 * DESIGN.md reading G25):
 *   tri_flags = 0                      lower, diagonal last -- identical to
 *                                      sptrsv_analyse_csr.
 *   SPTRSV_TRI_UPPER                   upper: per row strictly increasing
 *                                      columns, all >= i, column i FIRST,
 *                                      val[rowptr[i]] = U_ii != 0; solved by
 *                                      backward substitution
 *                                      x_i = (b_i - sum_{j>i} U_ij x_j) / U_ii.
 *   SPTRSV_TRI_UNIT_DIAG (| UPPER)     unit diagonal: no stored diagonal (a
 *                                      stored column i is an error), all
 *                                      entries strictly below (above) the
 *                                      diagonal, x_i = b_i - sum_j T_ij x_j.
 * Errors: other flag bits -> INVALID_ARG; an entry on the wrong side of the
 * diagonal (or a stored diagonal under UNIT_DIAG) -> SPTRSV_ERR_NOT_LOWER; a
 * missing / misplaced diagonal -> MISSING_DIAG; as sptrsv_analyse_csr
 * otherwise (lowest offending row wins).  Same ownership and synchronisation
 * as sptrsv_analyse_csr.
 * A handle with tri_flags != 0 runs, for an all-thread-level plan, the LEAN
 * engine or -- when >= 1/4 of its dependencies fall inside their own 32-row
 * group of logical rows (grids, chains) -- the CHAIN engine; a plan with
 * warp-level rows runs k_solve_tri_warp (one warp per long row, 32-row thread
 * groups for the rest).
 * Upper rows are taken in reverse order behind the same start ticket, so the
 * ticket order is a topological order.  Each row's off-diagonals are summed
 * earliest-solved first: ascending column (lower), descending column (upper).
 * sptrsv_solve, sptrsv_solve_multi (column by column), sptrsv_solve_host,
 * sptrsv_get_indegree, sptrsv_check and the
 * options work as for lower handles (ENGINE: 3 LEAN and 7 CHAIN are honoured
 * for all-thread-level plans, 8 SMALL for systems that fit one CTA);
 * sptrsv_levels and VARIANT != 0 return SPTRSV_ERR_INVALID_ARG.  Thread-level rows are bit-exact with that fp64
 * substitution (one rounded multiply and add each); warp rows are within the
 * warp-mode bound, as for lower handles.  sptrsv_info.engine: 3 LEAN, 6 warp,
 * 7 CHAIN, 8 SMALL (bit-exact: every row is thread-level there), 9 LEANP.
 */
int sptrsv_analyse_csr_ex(int32_t n, const int32_t *rowptr, const int32_t *colidx,
                          const double *val, int32_t tri_flags, sptrsv_handle_t *out);

/*
 * sptrsv_analyse_csr_batch -- a BATCH of independent systems (the
 * C5 batch of BASELINE configs[4]) as ONE handle, so that a solve is one launch
 * over all of them: the block-diagonal matrix diag(L_0, ..., L_{nsys-1}), each
 * block the paper's problem (Alg.5) on its own rows.
 *   nsys     number of systems (>= 1).
 *   n        HOST array [nsys]: rows of each system (>= 0).
 *   rowptr, colidx, val
 *            HOST arrays [nsys] of DEVICE pointers to each system's CSR, in the
 *            layout of sptrsv_analyse_csr (val / colidx may be NULL for a
 *            system with no entries, unit-diagonal forms only).
 *   tri_flags as sptrsv_analyse_csr_ex, for every system.
 * The library copies the systems into one handle-owned concatenation (rowptr
 * shifted by the entries, colidx by the rows before each system; freed by
 * sptrsv_destroy; the caller's arrays are not kept), then analyses it as
 * sptrsv_analyse_csr_ex does (same validation codes, row indices of the
 * concatenation).  Solves take the concatenated b / x: system s occupies rows
 * n[0] + ... + n[s-1] onward.  Synchronous.  Measured:
 * one launch over 2 C5 systems beats 2 launches; over 8 the ready words
 * outgrow the persisting L2 window and separate launches win -- group systems
 * by what the window holds.
 */
int sptrsv_analyse_csr_batch(int32_t nsys, const int32_t *n, const int32_t *const *rowptr,
                             const int32_t *const *colidx, const double *const *val, int32_t tri_flags,
                             sptrsv_handle_t *out);

/*
 * sptrsv_solve -- one solve L x = b (Alg.5), enqueued on
 * `stream`; asynchronous, never synchronises the host.  Exactly ONE kernel
 * launch (the per-solve flag reset of Alg.5 l.2 is an epoch bump done inside
 * the kernel), so it is CUDA-graph capturable.
 *   b  device, double[n], read-only.   x  device, double[n], fully overwritten.
 *   b and x must not alias.  Solves through one handle are ordered on one
 *   stream; concurrent solves with the same handle on different streams are
 *   undefined (shared flags).  Distinct handles are independent.
 * Returns launch errors only; a watchdog timeout is reported by sptrsv_check.
 */
int sptrsv_solve(sptrsv_handle_t h, const double *b, double *x, sptrsv_stream_t stream);

/*
 * sptrsv_solve_multi -- L X = B for nrhs right-hand sides at once (SURVEY row
 * f1; "multiple right-hand sides [21]"): one dependency hop per
 * row serves all nrhs solves.  Row-major: B[i*ldb + r], X[i*ldx + r],
 * 1 <= nrhs <= 32, ldb, ldx >= nrhs; B and X device, must not alias.  Same
 * protocol option and options as sptrsv_solve; asynchronous, one launch.
 * Each component (i, r) has its own ready word, so the handle keeps
 * n * nrhs of them (allocated on first use).  Handles whose solve runs the
 * CHAIN engine, and upper / unit-diagonal handles, solve column by column
 * instead (gather, sptrsv_solve, scatter per column, on `stream`): their
 * in-register chains beat one shared hop per row.
 */
int sptrsv_solve_multi(sptrsv_handle_t h, const double *B, double *X, int32_t nrhs, int64_t ldb, int64_t ldx,
                       sptrsv_stream_t stream);

/*
 * sptrsv_solve_host -- end-to-end convenience from host buffers; synchronises
 * `stream` before returning (the calling thread polls an event: it spins for
 * the duration of the solve rather than sleeping in a blocking sync).  b_host/x_host: host double[n].
 *   - Both pinned (page-locked, UVA-mapped; e.g. cudaHostAlloc or torch
 *     pin_memory) and the handle runs LEAN or LEANP: b is copied to device staging in
 *     about four chunks on a handle-owned second stream, each CTA of the solve
 *     waiting only for the chunk of its own rows, and every CTA writes its
 *     finished rows of x to x_host as one contiguous block -- both transfers
 *     overlap the solve (x also lands in handle-owned device staging).
 *     SPTRSV_OPT_HOST_IO selects the variants.
 *   - Both pinned and the handle runs SMALL: the kernel reads b from b_host
 *     and writes x to x_host through the UVA mapping (no copy launches).
 *   - Otherwise: b is copied to handle-owned device staging, solved, and x is
 *     copied back (cudaMemcpyAsync; pageable buffers are staged by the driver).
 */
int sptrsv_solve_host(sptrsv_handle_t h, const double *b_host, double *x_host,
                      sptrsv_stream_t stream);

/* sptrsv_destroy -- frees the handle's workspace (synchronises the device
 * first).  NULL is a no-op. */
int sptrsv_destroy(sptrsv_handle_t h);

int sptrsv_set_option(sptrsv_handle_t h, int key, int64_t value);
int sptrsv_get_option(sptrsv_handle_t h, int key, int64_t *value);

/* sptrsv_info -- sizes, plan and timing of the handle (host struct). */
int sptrsv_get_info(sptrsv_handle_t h, sptrsv_info *out);

/* sptrsv_get_indegree -- copies the in-degrees computed by analyse
 * (indeg[i] = number of stored off-diagonals of row i = dependencies of x_i,
 * PAPER.md:67-69) into device int32[n] `out_dev`, async on `stream`. */
int sptrsv_get_indegree(sptrsv_handle_t h, int32_t *out_dev, sptrsv_stream_t stream);

/*
 * sptrsv_levels -- diagnostic, not part of the solve: the level of every
 * component (level[i] = 0 without dependencies, else 1 + max
 * level of its dependencies) computed on the GPU with the same
 * synchronization-free flag protocol, plus the level-set histogram (Table 6
 * beta = n / nlevels).
 *   level_dev   device int32[n] or NULL.   counts_dev  device int32[n] or NULL;
 *   counts_dev[l] = components in level l for l < nlevels (entries >= nlevels
 *   are zero).  nlevels_host: host int32, receives max level + 1.
 * Synchronises `stream`.
 */
int sptrsv_levels(sptrsv_handle_t h, int32_t *level_dev, int32_t *counts_dev,
                  int32_t *nlevels_host, sptrsv_stream_t stream);

/* sptrsv_set_trace -- diagnostic: while trace_dev (device uint64[3n]) is set,
 * every solve writes the %globaltimer (ns) at which x_i was published into
 * trace_dev[i], and for thread-level rows the time row i consumed its last
 * dependency into trace_dev[n + i] and the time its solve loop started (data
 * loaded) into trace_dev[2n + i] -- the critical path, row by row.  NULL turns
 * it off. */
int sptrsv_set_trace(sptrsv_handle_t h, uint64_t *trace_dev);

/* sptrsv_check -- synchronises `stream`, returns SPTRSV_ERR_TIMEOUT if the
 * watchdog fired in any solve since the last check, SPTRSV_ERR_STALE_LAUNCH if
 * a stale graph launch was refused, else OK.  Clears the condition: the next
 * solve re-zeroes the ready words first, so it is correct again. */
int sptrsv_check(sptrsv_handle_t h, sptrsv_stream_t stream);

/*
 * sptrsv_flag_latency -- diagnostic microbenchmark on the current device: two
 * CTAs ping-pong `iters` times through the publish/consume pair the solve uses
 * and report the mean one-way hop in nanoseconds (t_hop of the critical-path
 * latency bound).  protocol: 0 = st.release flag / ld.acquire poll
 * + relaxed x load (the solve's protocol), 1 = relaxed poll + fence.acq_rel,
 * 2 = value-as-flag (x polled directly; ablation only); single-CTA probes:
 * 3 = dependent ld.relaxed.gpu chain (ns per L2 round trip), 4 = st x +
 * st.release flag pairs (ns per publish), 5 = dependent fp64 IEEE divisions,
 * 6 = dependent DFMA, 7 = shared-memory store->load round trip.  sm_mhz (host, may be NULL)
 * receives the SM clock seen during the probe (clock64 / globaltimer).
 * Synchronous.
 */
int sptrsv_flag_latency(int32_t iters, int32_t protocol, double *ns_per_hop, double *sm_mhz);

/*
 * sptrsv_hop_scan -- diagnostic, placement-controlled t_hop (the critical-path latency bound's
 * hop): one CTA per SM on the current device; the CTAs on SM sm_a (the
 * lowest SM id present) and on each other SM b ping-pong `iters` rounds through the solve's
 * publish / poll pair (protocol 0 FLAGS: st.release flag, ld.acquire poll + x load; 1 FUSED:
 * 16-byte epoch record, relaxed store / poll) and the mean one-way hop in ns is reported per b,
 * the fastest over 8 ready-word addresses 4 KB apart (the word's L2 slice, and its die, follow the
 * address).
 *   capacity    entries sm_b_out / ns_out can hold (host arrays).
 *   sm_a_out    host int32, receives sm_a.   count  host int32, receives the pairs measured.
 * Synchronous.  The two dies of a B200 show as two latency modes over b.
 */
int sptrsv_hop_scan(int32_t iters, int32_t protocol, int32_t capacity, int32_t *sm_a_out, int32_t *sm_b_out,
                    double *ns_out, int32_t *count);

const char *sptrsv_strerror(int status);
int sptrsv_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SPTRSV_H_ */
