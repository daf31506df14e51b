/*
 * spcg.h — C ABI of the B200-native SPCG library (libspcg.so).
 *
 * The method: Ma, Ahmad, Cheshmi, Sundar, Hall, "Sparsified Preconditioned
 * Conjugate Gradient Solver on GPUs" (SC'25).  "P:Lx-y" cites lines of
 * /root/reference/PAPER.md.  The library implements the pipeline of Figure 2
 * (P:L306-339): wavefront-aware sparsification (Algorithm 2) of
 * the SPD matrix A (Eq. 1) into Ahat, an ILU(0)/ILU(K) factorisation
 * M = {L, U} of Ahat (§3.3), and the iterative phase — PCG,
 * Algorithm 1 — whose SpMV uses the ORIGINAL A.
 *
 * Split of work:
 *   spcg_setup  (host C++, once)   validation, Algorithm 2, ILU(K) symbolic +
 *                                  numeric, level sets, device layouts, upload.
 *   spcg_solve  (device, sm_100a)  the whole of Algorithm 1 in one persistent
 *                                  cooperative CUDA kernel: SpMV (+ (p,w)),
 *                                  fused x/r update (+ ||r||^2), forward and
 *                                  backward SpTRSV (+ (r,z)), direction update,
 *                                  device-side alpha/beta and stopping test.
 *                                  No host round trip per iteration.
 *
 * Conventions (all calls):
 *   - Every function returns spcg_status_t; nothing throws or aborts across
 *     the ABI.  spcg_last_error() returns a thread-local detail string.
 *   - Matrices are 0-based CSR in host memory, FULL symmetric storage,
 *     int64 row pointers, int32 column indices (sorted, unique per row), f64.
 *   - Device vectors are plain device pointers (e.g. torch tensor data_ptr())
 *     on the handle's device; host vectors only where a flag says so.
 *   - Readings of passages the paper leaves open are the ones listed in
 *     DESIGN.md §2 and are selectable where cheap.
 */
#ifndef SPCG_H
#define SPCG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SPCG_ABI_VERSION 3

typedef int32_t spcg_status_t;
enum {
    SPCG_OK = 0,
    SPCG_NOT_CONVERGED = 1,     /* warning: x holds x_kmax (Alg. 1 line 17) */
    SPCG_ERR_INVALID_ARG = -1,
    SPCG_ERR_BAD_MATRIX = -2,   /* non-square, unsorted/duplicate cols, missing or <= 0 diagonal,
                                   non-finite value, not exactly (bitwise) symmetric, nnz >= 2^31 */
    SPCG_ERR_ZERO_PIVOT = -3,   /* u_ii == 0 or non-finite during ILU, or after rounding to fp32
                                   (row in setup info) */
    SPCG_ERR_BREAKDOWN = -4,    /* (p,w) <= 0 or a non-finite PCG scalar */
    SPCG_ERR_OOM = -5,
    SPCG_ERR_CUDA = -6,
    SPCG_ERR_INTERNAL = -7,
    SPCG_ERR_NO_DEVICE = -8     /* a device call on a host-only (device = -1) handle */
};

typedef struct spcg_handle_s* spcg_handle_t;

/* A (host memory, read only during spcg_setup; the library deep-copies it). */
typedef struct {
    int64_t n;
    int64_t nnz;
    const int64_t* row_ptr;   /* [n+1] */
    const int32_t* col_idx;   /* [nnz] */
    const double* val;        /* [nnz] */
} spcg_csr_t;

/* Sparsification (§3.2, Algorithm 2). */
enum {
    SPCG_DROP_NONE = 0,             /* Ahat = A: the unsparsified PCG baseline */
    SPCG_DROP_FIXED = 1,            /* Ahat = A - S_t with t = fixed_pct */
    SPCG_DROP_WAVEFRONT_AWARE = 2   /* Algorithm 2 over ratios_pct (default {10,5,1}) */
};
enum { SPCG_NORM_FRO = 0, SPCG_NORM_INF = 1,            /* reading A6 of ||Ahat||_2, ||S|| */
       SPCG_NORM_SPECTRAL = 2 };                        /* power method, 100 steps from (1..1) (host setup) */
enum { SPCG_DENOM_WA = 0, SPCG_DENOM_WAHAT = 1 };       /* reading A8: Eq. 7 vs Alg. 2 line 10 */

typedef struct {
    int32_t mode;               /* SPCG_DROP_* */
    double fixed_pct;           /* t for SPCG_DROP_FIXED, percent of nnz(tril A) (A1, A2) */
    int32_t n_ratios;           /* 1..8 */
    double ratios_pct[8];       /* applied in the given order (most aggressive first) */
    double tau;                 /* convergence threshold, default 1 */
    double omega_pct;           /* wavefront-reduction threshold, default 10 */
    int32_t norm_reading;       /* SPCG_NORM_* */
    int32_t reduction_denominator; /* SPCG_DENOM_* */
} spcg_drop_params_t;

/* Triangular-solve executors (the wavefront executor of §2). */
enum {
    SPCG_SPTRSV_AUTO = 0,
    SPCG_SPTRSV_LEVEL = 1,      /* level-scheduled: one grid barrier per wavefront */
    SPCG_SPTRSV_SYNCFREE = 2,   /* per-row ready flags, no level barriers */
    SPCG_SPTRSV_CHUNKED = 3,    /* rows partitioned into contiguous per-CTA chunks; intra-chunk
                                   dependencies through shared memory, cross-chunk through flags */
    SPCG_SPTRSV_RESIDENT = 4,   /* small systems (n <= SPCG_RESIDENT_MAX_N): one CTA holds every
                                   vector in shared memory; level-scheduled with CTA barriers */
    SPCG_SPTRSV_WCHAIN = 5      /* warp chains: rows split into chains (decoupled components or
                                   grid blocks), one warp walks a chain wavefront by wavefront with
                                   register (shuffle) handoffs; vectors in execution order */
};
#define SPCG_RESIDENT_MAX_N 4096

/* How the device loop of Algorithm 1 is orchestrated. */
enum {
    SPCG_EXEC_AUTO = 0,         /* = PERSISTENT */
    SPCG_EXEC_PERSISTENT = 1,   /* one persistent cooperative kernel per solve (device-side scalars) */
    SPCG_EXEC_GRAPH_WHILE = 2   /* a conditional-WHILE CUDA graph of per-phase kernels: NOT built in this
                                   library (a kernel launch per wavefront or phase is the design the
                                   persistent kernel replaces); setup returns SPCG_ERR_INVALID_ARG */
};

enum { SPCG_SETUP_HOST = 0, SPCG_SETUP_GPU = 1 };
enum { SPCG_FACTORS_F64 = 0, SPCG_FACTORS_F32 = 1 };

/* Device allocator hooks: when dev_alloc is set, every device buffer the handle owns
 * comes from dev_alloc(bytes, stream, ctx) and goes back through
 * dev_free(ptr, bytes, stream, ctx) (e.g. PyTorch's caching allocator; the Python
 * binding installs such a shim).  NULL = cudaMalloc / cudaFree.  A NULL return from
 * dev_alloc fails setup with SPCG_ERR_OOM.  The hooks are called from the thread that
 * calls spcg_setup / spcg_solve / spcg_destroy, never from device code, and must stay
 * valid (with ctx) until spcg_destroy returns. */
typedef void* (*spcg_dev_alloc_fn)(size_t bytes, void* stream, void* ctx);
typedef void (*spcg_dev_free_fn)(void* ptr, size_t bytes, void* stream, void* ctx);

typedef struct {
    int32_t device;             /* CUDA ordinal; -1 = host analysis only (export works, solve does not) */
    void* stream;               /* cudaStream_t for all device work (NULL = legacy default stream) */
    int32_t sptrsv;             /* SPCG_SPTRSV_* */
    int32_t parts;              /* CTAs of the persistent kernel (0 = auto from n and the SM count) */
    int32_t host_threads;       /* OpenMP threads for setup (0 = all) */
    int32_t exec;               /* SPCG_EXEC_* */
    spcg_dev_alloc_fn dev_alloc;
    spcg_dev_free_fn dev_free;
    void* alloc_ctx;
    double wide_min;            /* mean dependencies per row above which LEVEL/SYNCFREE use one warp per
                                   row (0 = default SPCG_WCAP = 8) */
    int32_t chunk_partition;    /* CHUNKED executor: -1 = inspector's choice (default), else force
                                   0 contiguous, 1 strided, 2 affinity, 3 components, 4 tiles */
    int32_t setup_device;       /* SPCG_SETUP_HOST (default) or SPCG_SETUP_GPU: validation, Algorithm 2,
                                   ILU(0) and the level sets on the GPU (NEXT-1; K = 0 only — K > 0 and
                                   K = -1 run on the host).  Products are bit-exact with the host setup
                                   except the Frobenius indicator values, which agree up to summation
                                   order (reading A6g) */
    int32_t factor_precision;   /* SPCG_FACTORS_F64 (default) or SPCG_FACTORS_F32 (NEXT-2, the paper's
                                   fp32 preconditioner): the ILU factor values are rounded to
                                   fp32 after the factorisation, M = fl32(L) fl32(U) applied in fp64
                                   (1/u_ii from the rounded u_ii); the warp-chain records then carry
                                   4-byte values.  Vectors and scalars stay fp64, so eps = 1e-8 holds */
    int32_t reserved[5];
} spcg_options_t;

typedef struct {
    double chosen_pct;          /* 0 = nothing dropped */
    int64_t m_t;                /* strictly-lower entries dropped (S has 2 m_t entries) */
    int64_t w_A;                /* wavefronts of tril(A) (Alg. 2 line 1) */
    int64_t w_Ahat;             /* wavefronts of tril(Ahat) */
    int32_t n_tried;
    double tried_pct[8];
    double indicator[8];        /* ||Ahat_t^-1|| ||S_t|| per tried ratio */
    int64_t tried_w[8];         /* -1 when the indicator test failed first */
    double tried_reduction_pct[8];
    int64_t n;
    int64_t nnz_A, nnz_Ahat, nnz_L, nnz_U;   /* nnz_L = strict lower, nnz_U includes the diagonal */
    int64_t levels_L, levels_U;
    int64_t zero_pivot_row;     /* -1 if none */
    double setup_ms_validate, setup_ms_sparsify, setup_ms_symbolic, setup_ms_numeric,
           setup_ms_layout, setup_ms_upload;
    int32_t sptrsv;             /* executor actually used */
    int32_t parts;              /* CTAs of the persistent kernel */
    int64_t device_bytes;       /* device memory held by the handle */
    double algo_bytes_per_iter; /* B_iter: what one iteration must move */
    double algo_flops_per_iter;
    int32_t partition;          /* CHUNKED: row partition the inspector chose — 0 contiguous, 1 strided,
                                   2 affinity, 3 components, 4 tiles; WCHAIN: 5
                                   components, 6 grid3d, 7 grid2d; -1 otherwise */
    int32_t chains;             /* WCHAIN: warp chains (0 otherwise) */
    int64_t positions;          /* WCHAIN: execution-order slots (32 x steps >= n) */
    int64_t chain_entries[4];   /* WCHAIN: dependencies read by shuffle / shared ring / global / flag */
    int32_t setup_device;       /* where validation .. ILU ran: SPCG_SETUP_HOST / SPCG_SETUP_GPU */
    double setup_ms_total;      /* spcg_setup wall time, entry to return */
    int32_t factor_precision;   /* SPCG_FACTORS_*: precision of the stored factor values */
    int32_t record_value_bytes; /* WCHAIN: bytes per stored factor value in the records (8 or 4) */
} spcg_setup_info_t;

typedef struct {
    int64_t iterations;         /* k: completed iterations when the test fired (or kmax) */
    double rnorm;               /* ||r_k||_2 of the recurrence residual */
    int32_t converged;
    spcg_status_t status;
    double iter_phase_ms;       /* device time of Alg. 1 from line 1 to exit (reading A19) */
    double total_ms;            /* including host<->device copies when SPCG_HOST_PTRS */
} spcg_solve_info_t;

/* Largest kmax a solve accepts (SPCG_ERR_INVALID_ARG above it): the device's
 * per-solve ready-flag epochs are 32-bit and advance by kmax + 3 per solve. */
#define SPCG_KMAX_LIMIT 1000000000LL

/* spcg_solve flags */
#define SPCG_USE_X0 0x1u        /* x holds the initial guess (default x0 = 0) */
#define SPCG_HOST_PTRS 0x2u     /* b and x are HOST pointers: copies happen inside the call */

/* spcg_export items (two-call size query: buf == NULL -> *bytes = size) */
enum {
    SPCG_EXPORT_AHAT_ROWPTR = 1, SPCG_EXPORT_AHAT_COL = 2, SPCG_EXPORT_AHAT_VAL = 3,
    SPCG_EXPORT_L_ROWPTR = 4, SPCG_EXPORT_L_COL = 5, SPCG_EXPORT_L_VAL = 6,
    SPCG_EXPORT_U_ROWPTR = 7, SPCG_EXPORT_U_COL = 8, SPCG_EXPORT_U_VAL = 9,
    SPCG_EXPORT_FILL_LEVEL = 10,            /* int32 level of fill per L+U entry, row-major */
    SPCG_EXPORT_LEVEL_L = 11, SPCG_EXPORT_LEVEL_U = 12,          /* int32 per-row level */
    SPCG_EXPORT_LEVELPTR_L = 13, SPCG_EXPORT_LEVELROWS_L = 14,   /* int64[w+1], int32[n] */
    SPCG_EXPORT_LEVELPTR_U = 15, SPCG_EXPORT_LEVELROWS_U = 16,
    SPCG_EXPORT_RHIST = 17      /* f64 ||r_k|| history of the last solve (k+1 values) */
};

/* ------------------------------------------------------------------ API */

int32_t spcg_abi_version(void);
const char* spcg_status_string(spcg_status_t s);
const char* spcg_last_error(void);

/* Defaults: mode WAVEFRONT_AWARE, ratios {10,5,1}, tau 1, omega 10,
 * Frobenius norms (A6), Eq. 7 denominator (A8). */
void spcg_drop_params_default(spcg_drop_params_t* p);
void spcg_options_default(spcg_options_t* o);

/* Builds the preconditioner of Fig. 2 and uploads everything the iterative
 * phase needs.  A: host CSR (validated; deep-copied).  drop: NULL = defaults.
 * K >= 0: ILU(K) level of fill (K = 0 is ILU(0)); K = -1: M = I (plain CG).
 * opt: NULL = defaults.  On error *out = NULL and the status says why. */
spcg_status_t spcg_setup(const spcg_csr_t* A, const spcg_drop_params_t* drop, int32_t K,
                         const spcg_options_t* opt, spcg_handle_t* out);

spcg_status_t spcg_get_setup_info(spcg_handle_t h, spcg_setup_info_t* info);

/* Runs Algorithm 1: x <- solution of A x = b, stopping when ||r_k||_2 < eps
 * (A13, strict) or after kmax iterations (A14).  eps = 0 is forced-k mode:
 * exactly kmax iterations, status SPCG_OK.  b, x: device pointers (length n,
 * 8-byte aligned) unless flags has SPCG_HOST_PTRS.  Enqueued on opt.stream;
 * returns after the stream work completes.  info may be NULL. */
spcg_status_t spcg_solve(spcg_handle_t h, const double* b, double* x, double eps, int64_t kmax,
                         uint32_t flags, spcg_solve_info_t* info);

/* NEXT-4: nrhs right-hand sides of the same system, each an
 * independent run of Algorithm 1 (own alpha, beta, stopping test; a converged one is
 * frozen while the others continue), with the matrix and factor streams read once per
 * group of up to 4.  B, X: device pointers, column-major n x nrhs
 * (column j = right-hand side j), x0 = 0, flags must be 0.  info: array of nrhs entries
 * (may be NULL); iter_phase_ms is the group's launch time.  Returns the worst status of
 * the right-hand sides.  Requires the warp-chain executor whose chains need only
 * shuffles (components / grid2d partitions without cross-chain terms), fp64 narrow
 * records (W <= 4) and the TMA SpMV: otherwise SPCG_ERR_INVALID_ARG with the reason. */
spcg_status_t spcg_solve_multi(spcg_handle_t h, const double* B, double* X, int32_t nrhs, double eps, int64_t kmax,
                               uint32_t flags, spcg_solve_info_t* info);

/* Asynchronous form of spcg_solve/* Asynchronous form of spcg_solve for running independent systems concurrently
 * (the C5 batch): enqueues Algorithm 1 on the handle's stream
 * and returns; b, x must be device pointers (SPCG_HOST_PTRS -> INVALID_ARG) and
 * stay valid until spcg_solve_wait(h, info) has returned, which synchronises
 * the stream and fills info exactly as spcg_solve does.  One solve in flight per
 * handle (a second spcg_solve_async before the wait -> INVALID_ARG).  Handles
 * set up on different streams run concurrently; each launch is cooperative, so
 * the caller keeps the CTAs (setup opt.parts) of the solves in flight on one
 * device within its SM count. */
spcg_status_t spcg_solve_async(spcg_handle_t h, const double* b, double* x, double eps, int64_t kmax,
                               uint32_t flags);
spcg_status_t spcg_solve_wait(spcg_handle_t h, spcg_solve_info_t* info);
/* Moves the handle's work to another cudaStream_t (a batch scheduler hands
 * systems to whichever lane is free).  The new stream waits on the device for
 * the work already queued on the old one (no host blocking); INVALID_ARG while
 * a solve is in flight. */
spcg_status_t spcg_set_stream(spcg_handle_t h, void* stream);

/* Single operators of the iterative phase on device vectors (length n), using
 * the same kernels as spcg_solve — for kernel-level parity tests:
 *   spmv:   w = A p          (A the ORIGINAL matrix), *pw = (p,w)
 *   lower:  y = L^-1 r       (unit lower factor)
 *   upper:  z = U^-1 y,      *rz = (r, z) when r != NULL
 *   precond: z = U^-1 L^-1 r (Alg. 1 line 13), *rz = (r, z) */
spcg_status_t spcg_apply_spmv(spcg_handle_t h, const double* p, double* w, double* pw);
spcg_status_t spcg_apply_lower(spcg_handle_t h, const double* r, double* y);
spcg_status_t spcg_apply_upper(spcg_handle_t h, const double* y, double* z, const double* r, double* rz);
spcg_status_t spcg_apply_precond(spcg_handle_t h, const double* r, double* z, double* rz);

/* Host copies of setup products (bit-exact parity tests). */
spcg_status_t spcg_export(spcg_handle_t h, int32_t what, void* buf, size_t* bytes);

void spcg_destroy(spcg_handle_t h);

/* Chain-floor calibration: the cost of each handoff a
 * wavefront executor can put on its critical path — P:L258-261 (Fig. 1 caption:
 * wavefront barriers "under-utilize GPU resources") — measured on `device`
 * with %globaltimer.  chain_floor = (levels_L + levels_U) x the handoff the
 * executor actually uses.  Times in ns; no handle needed; ~0.1 s of GPU time.
 * Errors: SPCG_ERR_INVALID_ARG (out == NULL), SPCG_ERR_CUDA (detail in
 * spcg_last_error()). */
typedef struct {
    double grid_sync_ns;        /* grid-wide barrier, one 256-thread CTA per SM (LEVEL, per wavefront) */
    double graph_kernel_ns;     /* kernel-to-kernel latency inside a CUDA graph (a launch per wavefront) */
    double flag_same_die_ns;    /* one-way release-store -> acquire-spin handoff, CTA pair on one die */
    double flag_cross_die_ns;   /* the same across the two dies */
    double syncthreads_ns;      /* __syncthreads, 256 threads */
    double cluster_sync_ns;     /* barrier.cluster arrive.release + wait.acquire, cluster of 2 */
    double sm_clock_mhz;        /* cudaDevAttrClockRate */
    int32_t sms;
    int32_t flag_pairs_near;    /* CTA pairs classified as same-die (of sms - 1) */
    double flag_relaxed_same_die_ns;   /* as flag_*, relaxed (volatile) accesses: the LL-flag handoff */
    double flag_relaxed_cross_die_ns;
} spcg_calib_t;
spcg_status_t spcg_calibrate(int32_t device, spcg_calib_t* out);

/* Ready-flag stress test (robustness of the "LL" flags of the sync-free, chunked and
 * warp-chain executors): a value is published as one 16-byte volatile
 * store {lo32, epoch, hi32, epoch} and accepted when both epochs read current, which
 * is sound only if each 8-byte half is observed whole.  Half of the SMs rewrite
 * `nslots` slots `rounds` times (one epoch per round), the other half poll them at
 * random throughout.  out[0] = torn reads (epochs agree, value halves from another
 * epoch: must be 0), out[1] = reads whose epochs differ (benign), out[2] = good reads.
 * Errors: SPCG_ERR_INVALID_ARG (out == NULL, sizes <= 0), SPCG_ERR_OOM, SPCG_ERR_CUDA. */
spcg_status_t spcg_ll_stress(int32_t device, int32_t nslots, int32_t rounds, uint64_t* out);

#ifdef __cplusplus
}
#endif
#endif /* SPCG_H */
