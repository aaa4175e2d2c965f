/*
 * rgsqr.h -- C-ABI of the B200-native recursive Gram-Schmidt QR library (librgsqr.so).
 *
 * Paper: S. Zhang, E. Baharlouei, P. Wu, "High Accuracy Matrix Computations on Neural
 * Engines: A Study of QR Factorization and its Applications", HPDC'20.  "P:Lnnn" cites a
 * line of PAPER.md; "reading #k" cites DESIGN.md's list of interpretations.
 *
 * Conventions (all entry points)
 *   - Every matrix is COLUMN-MAJOR fp32: element (i, j) of X with leading dimension ldx is
 *     X[i + j*ldx]; ldx >= rows.  Vectors are contiguous.
 *   - Data pointers may be DEVICE pointers (e.g. torch CUDA tensors; the call is then
 *     asynchronous on the handle's stream apart from the final status check) or HOST
 *     pointers (pageable or pinned; the library stages them through device workspace and the
 *     call returns when the results are back in host memory).  All matrix arguments of one
 *     call must be on the same side.  rgsqr_factor on PINNED host A, Q and R (single rank,
 *     reortho = 0) overlaps the copies with the factorization: A goes up in column chunks and
 *     Q / R columns come back as soon as their panel has run; the results are bit-identical to
 *     the device-pointer call.
 *   - The caller owns every input and output.  The library owns only the workspace inside the
 *     handle (grown lazily, freed by rg_destroy).
 *   - Return value: 0 = RG_OK; a NEGATIVE value -i means argument i (1-based, the handle is
 *     argument 1) is invalid (LAPACK `info` convention); positive values are the RG_* codes
 *     below.  rg_status_string() names them.
 *   - Row-sharded mode (after rg_comm_init): every rank passes its contiguous block of
 *     m_local rows (sum of m_local = m >= n); n and the options must match on all ranks and
 *     the call is collective.  R, x, S and V come back replicated; Q and U stay row-local.
 *
 * Thread-safety: a handle may be used by one host thread at a time.
 */
#ifndef RGSQR_H
#define RGSQR_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define RG_API __attribute__((visibility("default")))
#else
#define RG_API
#endif

typedef struct rg_handle_s* rg_handle;

enum {
    RG_OK = 0,
    RG_BREAKDOWN = 1,      /* zero or non-finite column norm: A is (numerically) rank deficient,
                              which the paper excludes; rg_last_info() gives the column */
    RG_NOT_CONVERGED = 2,  /* CGLS reached maxit (x holds the last iterate), or orthogonalize
                              reached max_passes above orth_tol (Q holds the last pass) */
    RG_NONFINITE = 3,      /* NaN/Inf in the input; rg_last_info() gives the column */
    RG_CUDA_ERROR = 4,     /* a CUDA runtime/driver call failed (handle stays usable if possible) */
    RG_NCCL_ERROR = 5,     /* NCCL missing or a collective failed */
    RG_NO_DEVICE = 6,      /* no sm_100 device / CUDA not initialisable */
    RG_ALLOC = 7           /* device or pinned host allocation failed */
};

/* Options.  rg_opts_default() fills the defaults listed here. */
typedef struct {
    int precision;  /* tensor-core operand type: 0 = fp16 (default), 1 = bf16 */
    int nb;         /* panel width of the recursion's base case, 1..32; 0 = auto (32).  With the
                       default nb = 32 and a single-GPU, non-split pass whose rows fit on chip
                       (m <= ~85K), the base case is a 64-column block factored by one leaf
                       kernel (CholQR2, fp64 Gram; reading #2) -- the same unique Q, R as two
                       32-column panels + K1 + K2 in exact arithmetic */
    int scale;      /* 1 = automatic power-of-two column scaling (default, section 3.5 P:L357-361,
                       reading #4); 0 = off */
    int reortho;    /* extra reorthogonalisation passes: for rgsqr_factor default 0; for
                       ls_solve_refined -1 = default: one split-precision pass, no reortho (reading #8) */
    int split;      /* 1 = 3 x 16-bit split-precision tensor-core GEMMs (reading #9), default 0;
                       orthogonalize always uses it for its refinement passes */
    int sync;       /* 1 (default) = synchronise at the end of the call and return breakdown /
                       non-finite status; 0 = fully asynchronous (status not checked) */
    int panel;      /* leaf panel algorithm: 0 = auto (default): CholQR2 with an fp64 Gram, falling
                       back on the device to the TSQR/MGS panel if a Cholesky pivot fails;
                       1 = TSQR/MGS only (eq 8 + Alg 2, the paper's panel) */
    int solver;     /* ls_solve_refined iteration: 0 = CGLS (default, Algorithm 3 as corrected by
                       reading #5), 1 = LSQR (same R preconditioner, same two passes over A
                       per iteration, same stopping test ||(A R^-1)^T r_k|| <= tol ||(A R^-1)^T b||) */
} rg_opts;

RG_API void rg_opts_default(rg_opts* o);

/* Create a handle bound to CUDA `device` and stream `cuda_stream` (a cudaStream_t; NULL =
 * the legacy default stream).  Returns RG_NO_DEVICE if the device is not sm_100. */
RG_API int rg_create(rg_handle* h, int device, void* cuda_stream);
RG_API int rg_set_stream(rg_handle h, void* cuda_stream);
RG_API int rg_destroy(rg_handle h);
RG_API const char* rg_status_string(int status);
/* Column index attached to the last RG_BREAKDOWN / RG_NONFINITE status (-1 if none). */
RG_API int64_t rg_last_info(rg_handle h);
/* Number of library kernels launched by the last API call on this handle (a CUDA-graph replay
 * counts the kernels it contains). */
RG_API int64_t rg_last_launches(rg_handle h);
/* Build identity, e.g. "rgsqr sm_100a tcgen05"; never NULL. */
RG_API const char* rg_version(void);

/* ---- row-sharded multi-GPU mode (the row split of eq 8) ----------
 * Each rank holds a contiguous block of rows; the collectives combine only small pieces (column
 * norms, the K1 blocks R12, the panel Gram matrices or TSQR R factors, CGLS vectors).  At most
 * RG_MAX_RANKS ranks (one 8-GPU node; the TSQR panel stacks <= 8 32 x 32 R factors).
 * Three ways to attach a handle to a group (each replaces the previous one and drops the
 * handle's cached plans):
 *   rg_comm_init  -- the library creates its own NCCL communicator from a ncclUniqueId that
 *                    rg_comm_unique_id wrote on the root rank (broadcast it, e.g. with
 *                    torch.distributed); destroyed with the handle.  nranks == 1 is allowed.
 *   rg_set_comm   -- use a CALLER-OWNED ncclComm_t (e.g. torch.distributed's); NULL detaches
 *                    (back to single-GPU mode).  The communicator must come from the same
 *                    libnccl the library loaded (rg_nccl_load with that path) and outlive the
 *                    handle's use of it.
 *   rg_set_vcomm  -- in-process "virtual ranks": P handles on ONE device share a group made by
 *                    rg_vgroup_create; each rank's API call must run on its own host thread,
 *                    concurrently.  Collectives are a host rendezvous + a fixed-order reduction
 *                    kernel; plans run eagerly (no CUDA graphs).  For testing the row-sharded
 *                    branches on one GPU; a rank that never arrives makes its peers fail with
 *                    RG_NCCL_ERROR after 120 s.
 * NCCL is loaded at run time (dlopen) from `nccl_path` (NULL = "libnccl.so.2").
 * Errors: -3 rank outside [0, nranks), -4 nranks outside [1, RG_MAX_RANKS]; rg_set_vcomm -2 the
 * group was created on another device; rg_vgroup_destroy -1 while handles are attached. */
#define RG_MAX_RANKS 8
RG_API int rg_nccl_load(const char* nccl_path);
RG_API int rg_comm_unique_id(void* id128);
RG_API int rg_comm_init(rg_handle h, const void* id128, int rank, int nranks);
RG_API int rg_set_comm(rg_handle h, void* nccl_comm, int rank, int nranks);
RG_API int rg_vgroup_create(void** group, int nranks);   /* on the current CUDA device */
RG_API int rg_vgroup_destroy(void* group);
RG_API int rg_set_vcomm(rg_handle h, void* group, int rank);

/* ---- rgsqr_factor: A = Q R (Algorithm 1) -------------------------------------
 * A (m_local x n, lda) is not modified unless Q aliases it (Q == A and ldq == lda: in place).
 * Q (m_local x n, ldq): orthonormal columns.  R (n x n, ldr): upper triangular with
 * positive diagonal, strictly-lower part zeroed, replicated on all ranks.
 * Recursive trailing updates R12 = Q1^T A2 and A2 -= Q1 R12 on tcgen05 tensor cores with
 * 16-bit operands and fp32 accumulation.  Base case (reading #2, #20): 64-column
 * leaves factored by CholQR2 with an fp64 Gram (rows resident on chip, m <= ~85K rows), else
 * 32-column CholQR2 panels (fused or streaming); opts->panel = 1 selects the paper's fp32
 * TSQR/MGS panel of eq 8 / Alg 2, which is also the automatic fallback when a
 * Cholesky pivot fails.  Requires m (global) >= n >= 1.
 * Errors: -2 m_local < 1 (or m < n single-GPU), -3 n < 1, -4 A NULL, -5 lda < m_local,
 * -6 Q NULL, -7 ldq < m_local, -8 R NULL, -9 ldr < n; RG_BREAKDOWN, RG_NONFINITE. */
RG_API int rgsqr_factor(rg_handle h, int64_t m_local, int64_t n, const float* A, int64_t lda, float* Q, int64_t ldq,
                 float* R, int64_t ldr, const rg_opts* opts);

/* ---- orthogonalize: Q with orthonormal columns spanning A (section 3.3) --------
 * A (m_local x n, lda) is overwritten by Q.  One RGSQR pass, then while the orthogonality
 * estimate ||I - Q^T Q||_F > orth_tol and passes < max_passes: [Q2, R2] = RGSQR(Q) with the
 * split-precision GEMMs (reading #9) and R <- R2 R ("twice is enough").
 * Tall blocks (n <= 256, rows beyond the on-chip leaf, e.g. config 4; every rank must agree when
 * row-sharded): each pass is one CholQR pass over the whole block on the tensor cores (reading
 * #33: split-16-bit Gram with fp64 column norms, n x n Gram allreduce when row-sharded, Cholesky
 * of the equilibrated Gram, in-place X <- X R^-1); a pass whose Cholesky fails or whose
 * equilibrated kappa_F(R) exceeds 32 n leaves A untouched and runs the RGSQR pass instead
 * (RGSQR_TALL=0 / 1 forces the path off / on).
 * R (n x n, ldr) receives the accumulated triangular factor if non-NULL.  passes_out: number
 * of passes run; orth_est_out: final ||I - Q^T Q||_F -- on the tall path computed exactly (in the
 * split Gram's precision) from the Gram of Q, which is also the next pass's Gram; otherwise a
 * Hutchinson estimate with 8 fixed Gaussian probes (E||M g||^2 = ||M||_F^2; within a few % of the
 * exact value).  orth_tol <= 0 means "run exactly max_passes passes".
 * Errors: -2..-6 as above (A is arg 4, lda arg 5, R arg 6, ldr arg 7 (< n with R non-NULL)),
 * -9 max_passes < 1; RG_NOT_CONVERGED if the final estimate is above orth_tol > 0. */
RG_API int orthogonalize(rg_handle h, int64_t m_local, int64_t n, float* A, int64_t lda, float* R, int64_t ldr,
                  double orth_tol, int max_passes, int* passes_out, double* orth_est_out, const rg_opts* opts);

/* ---- ls_solve_refined: x = argmin ||A x - b||_2 (eq 1; b in R^m, reading #14) ----
 * QR preconditioner (reading #8): by default (opts->reortho = -1) one RGSQR pass with split-
 * precision (3 x 16-bit) K1 / K2, whose R leaves kappa(A R^-1) ~ 1; opts->reortho >= 0 runs
 * RGSQR + that many reortho passes in opts->split precision.  Then CGLS preconditioned on the
 * right by R (Algorithm 3 as corrected by reading #5): vectors, reductions and scalars in
 * fp64, A read as fp32 (reading #7).  Stops when ||s_k|| <= tol ||s_0|| (reading #6) or after
 * maxit iterations.  b: m_local fp32; x: n fp64 (replicated).  iters_out / relres_out
 * (||s_k||/||s_0||) may be NULL.  Errors: -4 A NULL, -5 lda, -6 b NULL, -7 x NULL,
 * -8 tol < 0, -9 maxit < 0; RG_NOT_CONVERGED, RG_BREAKDOWN, RG_NONFINITE. */
RG_API int ls_solve_refined(rg_handle h, int64_t m_local, int64_t n, const float* A, int64_t lda, const float* b,
                     double* x, double tol, int maxit, int* iters_out, double* relres_out, const rg_opts* opts);

/* ---- lowrank_approx: A ~ U diag(S) V^T of rank `rank` (section 3.4; config 5) ---
 * Randomized range finder with RGSQR orthonormalisation (reading #17): Omega (n x l,
 * l = rank + oversample) ~ N(0,1) from Philox4x32-10 keyed by `seed`,
 * Y = A Omega, `power_iters` rounds of Z = A^T Q, Q_z = RGSQR(Z), Y = A Q_z, Q = RGSQR(Y);
 * B^T = A^T Q, [Q_b, R_b] = RGSQR(B^T), R_b = U_b S V_b^T (one-sided Jacobi),
 * U = Q V_b(:, 1:rank), V = Q_b U_b(:, 1:rank), S descending.
 * U: m_local x rank (ldu), S: rank, V: n x rank (ldv).
 * Errors: -4 A NULL, -5 lda, -6 rank < 1 or rank + oversample > n, -7 oversample < 0,
 * -8 power_iters < 0, -10 U NULL, -11 ldu, -12 S NULL, -13 V NULL, -14 ldv < n. */
RG_API int lowrank_approx(rg_handle h, int64_t m_local, int64_t n, const float* A, int64_t lda, int rank, int oversample,
                   int power_iters, uint64_t seed, float* U, int64_t ldu, float* S, float* V, int64_t ldv,
                   const rg_opts* opts);

/* ---- lowrank_qrsvd: deterministic QR-SVD low rank of a tall-skinny A (section 3.4) --
 * A = Q R (one RGSQR pass, no reorthogonalisation: "the roundoff errors in RGSQRF is insignificant"
 * next to the truncation error), R = U_R S V_R^T (one-sided Jacobi in fp64 on the n x n R),
 * A_r = Q U_R(:, 1:r) S_r V_R(:, 1:r)^T (Table 4).  U: m_local x rank (ldu, row-local in
 * row-sharded mode), S: rank (descending), V: n x rank (ldv, replicated).  Workspace: an m_local x n
 * fp32 Q plus its two 16-bit images and n x n fp64 Jacobi matrices.  Requires m (global) >= n,
 * n <= 4096.  Errors: -2 m_local, -3 n, -4 A NULL, -5 lda, -6 rank outside [1, n], -7 U NULL,
 * -8 ldu, -9 S NULL, -10 V NULL, -11 ldv < n; RG_BREAKDOWN, RG_NONFINITE. */
RG_API int lowrank_qrsvd(rg_handle h, int64_t m_local, int64_t n, const float* A, int64_t lda, int rank, float* U,
                         int64_t ldu, float* S, float* V, int64_t ldv, const rg_opts* opts);

/* ---- profiling (bench.py's roofline) -------------------------------------------------------
 * When enabled, each kernel class is bracketed by CUDA events on the handle's stream and the
 * per-class device time / launch count / algorithmic work accumulate until reset.
 * Classes: 0 = K2 update GEMM, 1 = K1 projection GEMM (+ split-K reduce), 2 = panel,
 * 3 = scale/cast, 4 = CGLS passes, 5 = other. */
RG_API int rg_profile_enable(rg_handle h, int enable);
RG_API int rg_profile_reset(rg_handle h);
RG_API int rg_profile_get(rg_handle h, int cls, double* ms, int64_t* launches, double* flops, double* bytes);

/* ---- generator access for parity tests -----------------------------------------------------
 * The seeded Gaussian stream behind lowrank_approx's Omega (seed = its `seed`) and the
 * orthogonality probes: element e takes Philox4x32-10 call e >> 1 with counter
 * {call lo32, call hi32, 0, 0} and key {seed lo32, seed hi32}; words (0, 1) for even e, (2, 3)
 * for odd e give u1 = (w_a + 1) 2^-32, u2 = w_b 2^-32, z = sqrt(-2 ln u1) cos(2 pi u2) (fp64).
 * rg_debug_philox writes the 4 raw words of calls 0 .. ncalls-1 (4 * ncalls uint32, DEVICE
 * pointer); rg_debug_gaussian writes z for e = 0 .. n-1 (n doubles, DEVICE pointer).  Both
 * synchronise.  Errors: -2 negative count, -4 pointer NULL or not device memory. */
RG_API int rg_debug_philox(rg_handle h, int64_t ncalls, uint64_t seed, uint32_t* words);
RG_API int rg_debug_gaussian(rg_handle h, int64_t n, uint64_t seed, double* out);

#ifdef __cplusplus
}
#endif
#endif /* RGSQR_H */
