/*
 * bsolve.h -- C ABI of the B200-native batched sparse iterative solver.
 *
 * What it computes (per system i of a batch, independently):
 *   x_i ~= A_i^{-1} b_i by Algorithm 1 of Kashi et al., IPDPS 2022
 *   (Sec. IV-D): BiCGSTAB (van der Vorst [18],
 *   PAPER.md:1240-1243) right-preconditioned with scalar Jacobi
 *   D_i^{-1} = diag(A_i)^{-1}, stopping each
 *   system on its own when the residual 2-norm falls below
 *   tau.  All A_i share ONE sparsity pattern
 *   (BatchCsr/BatchEll, Sec. IV-A); only values differ.
 *   The readings of the garbled/silent points of Alg. 1 are DESIGN.md R1-R19.
 *
 * Conventions for every entry point
 *   - Return value: BSOLVE_OK (0) or a negative bsolve_error code.  No C++
 *     exception ever crosses this ABI.  On error, bsolve_last_error() returns
 *     a thread-local, human-readable message.
 *   - Argument validation happens before any CUDA call, synchronously.
 *   - "device" pointers are CUDA device (or managed) memory of the handle's
 *     device, 8-byte aligned for double; "host" pointers are ordinary host
 *     memory (pinned memory makes bsolve_run_host faster but is optional).
 *   - Asynchronous entry points (bsolve_run, bsolve_spmv, bsolve_csr_to_ell)
 *     only enqueue work on `stream` (a cudaStream_t; NULL = legacy default
 *     stream) and never synchronise it.  Numerical outcomes are per system
 *     and land in iters/resnorm/status on that stream; non-convergence is NOT
 *     an error return.
 *   - A handle may be used from one host thread / stream at a time.
 *   - Everything is fp64 (the paper's precision: LAPACK dgbsv, FP64 peaks in
 *     Table I, tol 1e-10).
 */
#ifndef BSOLVE_H
#define BSOLVE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---------------------------------------------------------------- codes -- */
typedef enum bsolve_error {
  BSOLVE_OK = 0,
  BSOLVE_ERR_INVALID = -1,     /* bad argument: NULL, n<=0, batch<0, tol<0 or
                                  NaN, maxiter<0, wrong device, bad options    */
  BSOLVE_ERR_PATTERN = -2,     /* row_ptr not monotone/not starting at 0,
                                  column out of range, duplicate or unsorted
                                  column, missing diagonal entry              */
  BSOLVE_ERR_UNSUPPORTED = -3, /* valid request this build cannot run, e.g.
                                  forced SMEM placement that does not fit,
                                  row longer than 32 entries                  */
  BSOLVE_ERR_CUDA = -4,        /* a CUDA runtime call failed (message has it) */
  BSOLVE_ERR_NOMEM = -5        /* host or device allocation failed           */
} bsolve_error;

/* Layout of the per-system `values` array (Fig. 3). */
enum {
  BSOLVE_FMT_AUTO = 0, /* resolves to ELL                                      */
  BSOLVE_FMT_CSR = 1,  /* values[i*nnz + e]: entry e in the CSR order of
                          (row_ptr, col_idx)  (BatchCsr)     */
  BSOLVE_FMT_ELL = 2   /* values[i*W*n + k*n + r]: slot k of row r, column-
                          major (BatchEll).  W =
                          max entries per row (bsolve_info.ell_width).  WHICH
                          entry of row r sits in slot k is chosen by the
                          handle (bank-conflict-free gathers, DESIGN.md
                          "ELL slot map") and published by bsolve_ell_map;
                          bsolve_csr_to_ell converts CSR-ordered values.
                          Padding slots MUST hold 0.0.                        */
};

/* Where the matrix values live while a system iterates (PAPER.md:708-721,
 * 738-813: the paper's automatic shared-memory configuration). */
enum {
  BSOLVE_PLACE_AUTO = 0,   /* CLUSTER for large 9-point stencils, else SMEM
                              if one system's values fit, else STREAM         */
  BSOLVE_PLACE_SMEM = 1,   /* staged once into shared memory by TMA bulk copy */
  BSOLVE_PLACE_STREAM = 2, /* re-read from global memory (L2/L1) every SpMV   */
  BSOLVE_PLACE_REGS = 3,   /* persistent kernel, one CTA per SM: values staged by
                              TMA, then held in REGISTERS for the whole solve;
                              the next system's TMA overlaps the current one
                              (ELL, 9 entries per row, even n <= 1024)        */
  BSOLVE_PLACE_CLUSTER = 4, /* one system per thread-block cluster of C CTAs
                              (1024 rows each, C <= 8) exchanging halo rows
                              and reduction partials through distributed
                              shared memory; 9-point stencils, even
                              1024 < n <= 8192 (AUTO picks it there)         */
  BSOLVE_PLACE_TMEM = 5    /* values staged by TMA, then held in TENSOR MEMORY
                              (tcgen05.st / tcgen05.ld, each thread its own
                              TMEM lane); SMEM carries only the gathered
                              vector; 9-point stencils, n <= 1024             */
};

/* Stopping criterion (R5). */
enum {
  BSOLVE_STOP_REL_B = 0, /* ||r||_2 < tol * ||b||_2  (default)                */
  BSOLVE_STOP_ABS = 1    /* ||r||_2 < tol            (paper's experiments,
                            PAPER.md:869-870)                                  */
};

/* Krylov solver ("several preconditionable iterative
 * solvers"; BiCGSTAB is the paper's method, SURVEY.md 8(f) f3 the others). */
enum {
  BSOLVE_SOLVER_BICGSTAB = 0, /* Algorithm 1               */
  BSOLVE_SOLVER_GMRES = 1     /* restarted right-preconditioned GMRES(m)
                                 (Saad Alg. 6.9/6.11/9.5); every cycle starts
                                 from the true residual; 2D stencil patterns
                                 with n <= 1024 (line-tiled TMEM plan)        */
};
#define BSOLVE_MAX_RESTART 7

/* Preconditioner M^-1 applied on the right. */
enum {
  BSOLVE_PREC_JACOBI = 0, /* d_i = 1 / a_ii (a zero diagonal gives 1)          */
  BSOLVE_PREC_NONE = 1,   /* d_i = 1                                           */
  BSOLVE_PREC_BLOCK_JACOBI = 2 /* M = block diagonal of A with
                              blocks of 8 consecutive rows, each solved exactly
                              (R30).  BiCGSTAB on the line-tiled TMEM
                              plans only (2D 9-point stencils, where every block
                              is tridiagonal: grid width 9..120 with n <= 1024,
                              or width 64 with 1024 < n <= 8192 on the cluster
                              plan); UNSUPPORTED elsewhere                    */
};

/* Per-system outcome written to status[] (R10). */
enum {
  BSOLVE_SYS_CONVERGED = 0, /* final TRUE ||b - A x||_2 < tau                 */
  BSOLVE_SYS_MAXITER = 1,   /* maxiter iterations done without convergence    */
  BSOLVE_SYS_BREAKDOWN = 2, /* a BiCGSTAB denominator was 0 or non-finite;
                               x is the last finite iterate                   */
  BSOLVE_SYS_DIRECT = 3     /* direct_fallback: the iterative solve did not
                               converge (status 1 or 2) and x comes from the
                               banded LU (bsolve_banded_solve); resnorm is
                               its true residual, iters the iterative count   */
};

typedef struct bsolve_options {
  int format;              /* BSOLVE_FMT_*                 (default AUTO)     */
  int placement;           /* BSOLVE_PLACE_*               (default AUTO)     */
  int stop;                /* BSOLVE_STOP_*                (default REL_B)    */
  int true_residual_check; /* 1: recompute ||b - A x|| at exit and restart if
                              it is >= tau (R4); 0: trust the
                              recursive residual of Alg. 1  (default 1)       */
  int device;              /* CUDA device ordinal, -1 = current (default -1)  */
  int block_threads;       /* threads per CTA: 0 = auto, 128, 256 or 512
                              (default 0); 128 = 8 rows per thread (ELL) */
  int reg_slots;           /* with block_threads = 128 or the cluster plan:
                              off-diagonal ELL slots held in registers instead
                              of SMEM, 0, 2, 4, 6 or 8 (default 0 = planner's
                              choice: 4)                                      */
  int solver;              /* BSOLVE_SOLVER_* (default BICGSTAB)               */
  int precond;             /* BSOLVE_PREC_*   (default JACOBI)                 */
  int restart;             /* GMRES: Krylov steps per restart cycle m,
                              1 <= m <= BSOLVE_MAX_RESTART (default 7)        */
  int direct_fallback;     /* 1: after the iterative solve, every system whose
                              status is not CONVERGED is re-solved by the
                              banded LU on the same stream
                              and gets status DIRECT; a singular band keeps
                              the iterative result.  Two more launches per
                              bsolve_run (a device-side list of the failed
                              systems, one solve over that list); buffers
                              are allocated by bsolve_create.  Needs status
                              != NULL in bsolve_run (default 0)            */
} bsolve_options;

typedef struct bsolve_info {
  int n, nnz, batch;
  int ell_width;           /* W = max entries in a row                        */
  int format, placement;   /* resolved BSOLVE_FMT_* / BSOLVE_PLACE_*          */
  int block_threads;       /* CTA size used by the solve kernel               */
  int rows_per_thread;     /* rows each thread owns                           */
  int smem_bytes;          /* dynamic shared memory per CTA                   */
  int ctas_per_sm;         /* resident CTAs per SM                            */
  int num_sms;             /* SMs on the device                               */
  int grid;                /* CTAs launched per bsolve_run (REGS: persistent) */
  int kl, ku;              /* lower / upper bandwidth of the pattern          */
  int device;
  int kernel_mode;         /* 1 CSR column table, 2 ELL column table, 3 DIA:
                              ELL values whose slot k is column row + d_k in
                              every row (stencils; uniform gather offsets),
                              4 LINE: DIA on a 2D grid, each thread owns
                              consecutive grid rows (DESIGN.md Kernels 10)   */
  int cluster;             /* CTAs per system (PLACE_CLUSTER), else 0        */
  int solver, precond, restart; /* resolved BSOLVE_SOLVER_*, BSOLVE_PREC_*, m  */
  int banded_launches;     /* kernel launches of the last bsolve_banded_solve
                              (or direct-fallback) call: 2 per system chunk in
                              the split mode, 1 fused; 2 for a direct
                              fallback (compaction + fused solve); 0 before
                              the first                                      */
  int regs_per_thread;     /* registers of the solve kernel (TMEM plans), else 0 */
  int occupancy_api;       /* cudaOccupancyMaxActiveBlocksPerMultiprocessor for
                              it (TMEM plans; ctas_per_sm is computed from the
                              register, SMEM, thread and TMEM-column limits) */
  int line_width;          /* kernel_mode 4: the 2D grid width the line-tiled
                              kernel runs (a compile-time width: 31, 32, 64;
                              or any width <= 120 through the generic-width
                              instances), else 0                             */
  int line_generic;        /* 1: the generic-width instance (width mod 8 at
                              compile time, width / 8 at run time), else 0  */
  int max_active_clusters; /* PLACE_CLUSTER: cudaOccupancyMaxActiveClusters of
                              the cluster kernel (systems in flight), else 0 */
} bsolve_info;

typedef struct bsolve_plan *bsolve_handle; /* opaque; owns pattern + plan     */

/* Fill *opt with the defaults listed above. */
void bsolve_default_options(bsolve_options *opt);

/* Analyse one shared sparsity pattern and build a solve plan.
 *   out      [out] receives the handle (NULL on failure).
 *   n        rows (= columns) of every A_i, n >= 1.
 *   batch    number of systems each bsolve_run solves, batch >= 0.
 *   row_ptr  HOST, n+1 int32, row_ptr[0] = 0, non-decreasing.
 *   col_idx  HOST, row_ptr[n] int32, strictly increasing inside each row,
 *            every row containing its diagonal (Jacobi needs a_rr).
 *   opt      NULL for defaults.
 * The handle copies what it needs; the caller keeps ownership of the arrays.
 * Errors: INVALID, PATTERN, UNSUPPORTED, CUDA, NOMEM. */
int bsolve_create(bsolve_handle *out, int n, int batch, const int32_t *row_ptr,
                  const int32_t *col_idx, const bsolve_options *opt);

/* Solve all `batch` systems (one asynchronous kernel launch; 3 with
 * direct_fallback).
 *   values   DEVICE, batch * nnz (CSR) or batch * W * n (ELL) doubles.
 *   b        DEVICE, batch * n doubles (read only).
 *   x0       DEVICE, batch * n doubles, or NULL for the zero guess; may alias
 *            x (warm start "x in/out").
 *   tol      >= 0, finite.  maxiter >= 0 (0 returns x = x0, iters = 0).
 *   x        DEVICE, batch * n doubles (out).
 *   iters    DEVICE, batch int32 (out): executions of "v <- A p^" (R8).
 *   resnorm  DEVICE, batch doubles (out): final TRUE ||b - A x||_2, absolute.
 *   status   DEVICE, batch int8 (out) or NULL: BSOLVE_SYS_*.
 *   stream   cudaStream_t or NULL.
 * Caller owns all buffers; they must stay valid until the stream reaches
 * this work.  b = 0 under REL_B gives x = 0, iters = 0, CONVERGED. */
int bsolve_run(bsolve_handle h, const double *values, const double *b, const double *x0,
               double tol, int maxiter, double *x, int32_t *iters, double *resnorm,
               int8_t *status, void *stream);

/* Same computation with HOST buffers (same shapes as bsolve_run; x0 and
 * status may be NULL).  The library streams the batch through the device in
 * chunks: host->device copies, solve and device->host copies of successive
 * chunks overlap on internal streams.  Synchronous: returns when x, iters,
 * resnorm, status are written.  Pinned (page-locked) host memory is needed
 * for the copies to overlap; pageable memory works but serialises. */
int bsolve_run_host(bsolve_handle h, const double *values, const double *b, const double *x0,
                    double tol, int maxiter, double *x, int32_t *iters, double *resnorm,
                    int8_t *status);

/* Batched SpMV y_i = A_i x_i for `batch` systems (
 * the Fig. 7 microbenchmark).  values in the handle's
 * format; x, y DEVICE batch * n doubles (y must not alias x). Asynchronous. */
int bsolve_spmv(bsolve_handle h, const double *values, const double *x, double *y, int batch,
                void *stream);

/* Re-layout CSR-ordered values (batch * nnz) into the handle's ELL layout
 * (batch * W * n, zero padding).  DEVICE pointers, must not overlap.
 * Asynchronous.  Bit-exact: a pure permutation with zero fill. */
int bsolve_csr_to_ell(bsolve_handle h, const double *csr_values, double *ell_values, int batch,
                      void *stream);

/* Describe the plan (see bsolve_info). */
int bsolve_query(bsolve_handle h, bsolve_info *info);

/* Publish the handle's ELL slot map to HOST memory (either pointer may be
 * NULL, not both):
 *   cols[k*n + r]  column read by slot k of row r (W*n int32);
 *   src[k*n + r]   index e of the CSR entry (row_ptr/col_idx order) stored in
 *                  that slot, or -1 for a padding slot (value must be 0.0).
 * Every CSR entry appears in exactly one slot of its row. */
int bsolve_ell_map(bsolve_handle h, int32_t *cols, int32_t *src);

/* Host-only: the ELL slot map the library uses for a pattern, without a
 * handle or a GPU (same validation as bsolve_create).  *width receives W;
 * cols/src (W*n int32 each, may be NULL) as in bsolve_ell_map. */
int bsolve_ell_layout(int n, const int32_t *row_ptr, const int32_t *col_idx, int32_t *width,
                      int32_t *cols, int32_t *src);

/* Batched banded LU with partial pivoting and solve -- the GPU analogue of
 * LAPACK dgbsv, the paper's CPU solver for these systems (PAPER.md:97-99,
 * Sec. I; 556-559, Sec. III; 915-925, Sec. V-A).  For
 * every system i: P_i A_i = L_i U_i by dgbtf2's column order (pivot = FIRST
 * row of largest |a_kj| among rows j..j+kl), then x_i = U_i^-1 L_i^-1 P_i b_i
 * as in dgbtrs.  kl, ku are the pattern's bandwidths (bsolve_info.kl/ku).
 *   values  DEVICE, in the handle's format (as bsolve_run).
 *   b       DEVICE, batch * n doubles (read only).
 *   x       DEVICE, batch * n doubles (out; must not alias b).  Unspecified
 *           for a system with info > 0.
 *   info    DEVICE, batch int32 (out): 0, or j+1 for the first j with an
 *           exactly zero pivot u_jj (LAPACK convention: singular).
 *   ipiv    DEVICE, batch * n int32 (out) or NULL: 0-based row interchanged
 *           with row j at step j (ipiv[j] >= j).
 *   stream  cudaStream_t or NULL.  Asynchronous after the first call: per
 *           chunk of systems two kernel launches (factorisation writing U and
 *           y to the workspace, then the back substitution; bsolve_info.
 *           banded_launches reports the count of the last call).
 * The FIRST call (per handle) is synchronous host work: it builds and uploads
 * the banded pattern tables and allocates the workspace, n x (2 kb + 2)
 * doubles per system of a chunk (whole waves of resident CTAs, at most
 * ~8 GB), kb = max(kl, ku) rounded up to 4, 8, 16, 33 or 65.  With
 * direct_fallback the tables are built, and the fallback's own bounded
 * workspace (<= 256 MB) allocated, by bsolve_create; bsolve_run never
 * allocates.  Errors: INVALID (NULL / foreign pointers), UNSUPPORTED
 * (max(kl, ku) > 65, or a row with more entries than the instance has
 * loader lanes), NOMEM, CUDA. */
int bsolve_banded_solve(bsolve_handle h, const double *values, const double *b, double *x,
                        int32_t *info, int32_t *ipiv, void *stream);

/* bsolve_banded_solve with HOST buffers (values, b as for bsolve_run_host;
 * x: batch * n doubles out; info: batch int32 out).  The batch streams through
 * the device in chunks on the handle's 3 internal streams, copies of one chunk
 * overlapping the solve of another (pinned memory needed for the overlap).
 * Synchronous.  Errors as bsolve_banded_solve. */
int bsolve_banded_solve_host(bsolve_handle h, const double *values, const double *b, double *x,
                             int32_t *info);

/* Release the handle and its device memory.  NULL-safe; returns BSOLVE_OK. */
int bsolve_destroy(bsolve_handle h);

/* Message of the last non-OK return on the calling thread ("" if none). */
const char *bsolve_last_error(void);

/* Measure this device's shared-memory load bandwidth (bytes/s) with a
 * streaming LDS.128 kernel over all SMs; used as a measured roofline
 * denominator by bench.py.  Synchronous.  Writes *bytes_per_s and the SM
 * clock the kernel saw (*sm_hz, from clock64 over the event time). */
int bsolve_probe_smem_bandwidth(int device, double *bytes_per_s, double *sm_hz);

/* Measure this device's FP64 FMA throughput (flop/s, 2 per DFMA) with a
 * register-only DFMA loop over all SMs (8 independent chains per thread, 4
 * CTAs x 256 threads per SM): the measured FP64 roofline denominator of
 * bench.py.  Synchronous.  *sm_hz as above. */
int bsolve_probe_fp64(int device, double *flops_per_s, double *sm_hz);

#ifdef __cplusplus
}
#endif
#endif /* BSOLVE_H */
