// kernels.h -- internal launcher declarations shared by the .cu kernel files and the
// host driver (rgsqr.cpp).  Not part of the public C-ABI (include/rgsqr.h).
#pragma once
#include <cstddef>
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

#include <utility>

namespace rg {

// Programmatic dependent launch (PDL): every library kernel is launched with the
// programmatic-stream-serialisation attribute and starts with RG_PDL_ENTRY(), which lets the
// next kernel's launch overlap this one's tail and then waits (griddepcontrol.wait) for the
// previous grid to complete before touching memory.  Opt-in with RGSQR_PDL=1 (measured slower
// than plain graph edges for this kernel mix; kept for experiments).
#define RG_PDL_ENTRY()                                           \
    do {                                                         \
        asm volatile("griddepcontrol.wait;" ::: "memory");       \
        asm volatile("griddepcontrol.launch_dependents;" :::);   \
    } while (0)

bool pdl_enabled();

// Per-device properties of the CURRENT device (cached per device ordinal, thread-safe): one process
// may drive several GPUs (one handle per device, or in-process virtual ranks).
int dev_sms();              // multiprocessor count
int dev_smem_optin();       // cudaDevAttrMaxSharedMemoryPerBlockOptin
// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once per (device, kernel) and whenever a larger
// size is needed on that device; the attribute is per device context.
cudaError_t ensure_smem_attr(const void* kernel, size_t bytes);

// ---- tall.cu (one CholQR pass of a tall block, n <= 256, on tcgen05; reading #33)
size_t tall_ws_bytes();
double* tall_gram_buffer(void* ws);          // n x n fp64 Gram (allreduced in place when row-sharded)
int* tall_flag(void* ws);                    // nonzero after a failed pass (X untouched)
double* tall_kout(void* ws);                 // [kappa_F(R^), first failed pivot]
double* tall_dbg(void* ws);                  // [TL_N] tensor-core Gram diagonal (RGSQR_TALL_DEBUG)
// tmX: fp32 map of X (inner = rows, box 32 rows x 256 columns, no swizzle) or null (register-fed kernel)
cudaError_t launch_tall_gram(const float* X, int64_t ldx, int64_t m, int n, float sig, int bf16, void* ws, double* G,
                             cudaStream_t st, const CUtensorMap* tmX = nullptr);
cudaError_t launch_tall_orth(const double* G, int n, double sig, double* out, cudaStream_t st);
cudaError_t launch_tall_chol_apply(float* X, int64_t ldx, int64_t m, int n, const double* G, double sig_g, float sig_a,
                                   int bf16, double kappa_max, float* R, int64_t ldr, void* ws, cudaStream_t st);

template <typename... KArgs, typename... Args>
inline cudaError_t launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                            Args&&... args);

#define RG_LAUNCH(kern, grid, block, smem, st, ...)                                          \
    do {                                                                                     \
        cudaError_t _le = ::rg::launch_k(kern, dim3(grid), dim3(block), (size_t)(smem), st, __VA_ARGS__); \
        if (_le != cudaSuccess) return _le;                                                  \
    } while (0)

// kernel launches issued by this thread (bench.py "gpu_launches" claim)
extern thread_local long long g_launches;

// ---- scale.cu (section 3.5)
cudaError_t launch_colnorm(const float* A, int64_t lda, int64_t m, int n, double* partial, double* norm2,
                           cudaStream_t st);
cudaError_t launch_colscale(const double* norm2, int n, int do_scale, float* scale, int* status, int col0,
                            cudaStream_t st);
size_t colnorm_partial_doubles(int64_t m, int n);
cudaError_t launch_scale_cast(const float* A, int64_t lda, float* Q, int64_t ldq, uint16_t* Qh, uint16_t* Ql,
                              int64_t ldh, int64_t m, int n, const float* scale, int bf16, cudaStream_t st);
cudaError_t launch_unscale_r(float* R, int64_t ldr, int n, const float* scale, cudaStream_t st, int c0 = 0,
                             int nc = -1);

// ---- panel.cu (eq 8 + Alg 2)
struct PanelLaunch {
    float* Q;
    int64_t ldq;
    uint16_t* Qh;
    uint16_t* Ql;
    int64_t ldh;
    int64_t m;
    int nc;
    float* R;
    int64_t ldr;
    float* ws;
    int* counters;
    int distributed;
    int bf16;
    int col0;
    int* status;
    const int* guard;   // non-null: the kernels run only if *guard != 0 (CholQR2 fallback)
};
int panel_levels(int ntiles, int* lvl_n);
size_t panel_ws_floats(int64_t m);
size_t panel_counters(int64_t m);
cudaError_t launch_panel(const PanelLaunch& pl, cudaStream_t st);
cudaError_t launch_panel_apply(const PanelLaunch& pl, const float* Gq, cudaStream_t st);
cudaError_t launch_panel_stack(const float* Rall, int P, int nc, float* R, int64_t ldr, float* Qblocks, int* status,
                               int col0, const int* guard, cudaStream_t st);

// ---- panel_cholqr.cu (CholQR2, fp64 Gram)
struct CholqrLaunch {
    const float* P;
    int64_t ldp;
    float* Q;
    int64_t ldq;
    uint16_t* Qh;
    uint16_t* Ql;
    int64_t ldh;
    int64_t m;
    int nc;
    double* ws;     // cholqr_ws_doubles(m)
    int* counter;   // cholqr_counter_ints(m), zero-initialised, self-resetting
    int* fail;      // set on a failed pivot (guards the MGS fallback)
    float* R;
    int64_t ldr;
    int bf16;
    int (*allreduce_g)(double* G, void* ctx);  // non-null: multi-rank Gram allreduce (1024 doubles)
    void* ctx;
    unsigned long long cond;   // CUDA graph conditional handle set to 1 on a failed pivot (0: none)
    int* status;    // fused kernels report a numerical breakdown here (atomicMin col0 + j)
    int col0;       // global column index of the panel
    // fused single-panel kernel only: first apply Algorithm 1 line 9, P <- P - Q1 R12 (uh <= 64)
    const float* uq = nullptr;   // Q1, fp32 m x uh (ld uq_ld)
    int64_t uq_ld = 0;
    const float* ur = nullptr;   // R12, fp32 uh x nc (ld ur_ld)
    int64_t ur_ld = 0;
    int uh = 0;
};
size_t cholqr_ws_doubles(int64_t m);
size_t cholqr_counter_ints(int64_t m);
// True when the single-kernel path applies (rows per SM fit in shared memory; ncols 32 or 64).
bool cholqr_fused_fits(int64_t m, int ncols);
// *handles_failure = true: the launched kernel handles failed pivots itself (shifted CholQR3 +
// breakdown status); false: the caller must enqueue the guarded MGS/TSQR fallback kernels.
cudaError_t launch_panel_cholqr(const CholqrLaunch& L, bool* handles_failure, cudaStream_t st);
// Last recursion level (two 32-column panels, K1, K2) as one 64-column CholQR2 kernel on a
// 32 < nc <= 64 block: same Q and R in exact arithmetic; R written as the nc x nc block at L.R.
cudaError_t launch_panel_pair(const CholqrLaunch& L, cudaStream_t st);

// ---- leaf.cu (last recursion level: panel, K1, K2, panel in one cooperative kernel)
struct LeafLaunch {
    float* Q;          // nc block columns, in = P, out = Q (fp32, ldq)
    int64_t ldq;
    uint16_t* Qh;      // 16-bit shadow (hi) of Q, ldh
    uint16_t* Ql;      // lo part (split mode) or null
    int64_t ldh;
    int64_t m;
    int nc;            // 1..64: first panel min(32, nc) columns, second the rest
    float* R;          // nc x nc diagonal block of R (ldr)
    int64_t ldr;
    double* ws;        // leaf_ws_doubles()
    unsigned* bar;     // zero-initialised grid-barrier word
    int* status;
    int col0;
    int bf16;
    // prologue: Algorithm 1 lines 8-9 of the level above for this block, R_AB = Q_A^T P written
    // to R[-ph .. -1, 0 .. nc) (rows above the diagonal block), then P -= Q_A R_AB
    const uint16_t* pq = nullptr;   // Q_A 16-bit image (ld ldh, 16-byte aligned), null = none
    int ph = 0;                     // its columns, 1..64
};
bool leaf_fits(int64_t m);          // rows per SM fit in shared memory (and RGSQR_NO_LEAF unset)
bool leaf_prologue_fits(int64_t m); // ... and the 16-bit staging copy of the prologue's Q_A
size_t leaf_ws_doubles();
size_t leaf_stats_offset();   // doubles into the leaf workspace: 3 uint64 counters (launches, fast-Gram fallbacks, passes)
cudaError_t launch_leaf(const LeafLaunch& L, cudaStream_t st);

// ---- gemm_tc.cu (Alg 1 lines 8-9 on tcgen05)
cudaError_t launch_proj_gemm(int bn, bool split, int tiles_i, int tiles_j, int splits, const CUtensorMap& q1,
                             const CUtensorMap& a2, const CUtensorMap& q1_lo, const CUtensorMap& a2_lo, float* P,
                             int64_t ldp, int64_t p_stride, int kb_total, int kb_per_split, int bf16,
                             cudaStream_t st, int jfast = 0);
cudaError_t launch_update_gemm(int bn, bool split, int64_t m, int w, int h, const CUtensorMap& q1_mn,
                               const CUtensorMap& r12, const CUtensorMap& q1_mn_lo, const CUtensorMap& r12_lo,
                               float* C, int64_t ldc, void* Ch, void* Cl, int64_t ldh, int bf16, cudaStream_t st,
                               int overwrite = 0, const CUtensorMap* mc = nullptr, int h0 = 0);
// (mc: fp32 C, box 128 rows x 32 columns, no swizzle: K2 runs with the TMA epilogue.  h0: the
// 16-bit image of C is written for columns >= h0 only.)
cudaError_t launch_proj_reduce(const float* P, int64_t ldp, int64_t p_stride, int splits, int h, int w, float* R,
                               int64_t ldr, float* Rf, int64_t ldf, uint16_t* Rh, uint16_t* Rl, int64_t ldh, int bf16,
                               cudaStream_t st);
cudaError_t launch_proj_finish(const float* Rf, int64_t ldf, int h, int w, float* R, int64_t ldr, uint16_t* Rh,
                               uint16_t* Rl, int64_t ldh, int bf16, cudaStream_t st);

// ---- sgemm.cu (fp32 SIMT K1 / K2: the Figure 7 "no TensorCore" ablation, RGSQR_NO_TC=1)
size_t sgemm_tn_work_floats(int64_t m, int h, int w);
cudaError_t launch_sgemm_proj(const float* Q1, const float* A2, int64_t ld, int64_t m, int h, int w, float* R,
                              int64_t ldr, float* work, cudaStream_t st);
cudaError_t launch_sgemm_update(const float* Q1, const float* R12, int64_t ldr, float* A2, int64_t ld, int64_t m, int h,
                                int w, cudaStream_t st);

// ---- lowrank.cu
cudaError_t launch_cast_rows(const float* src, int64_t lds, int64_t rows, int cols, const float* rscale, uint16_t* hi,
                             uint16_t* lo, int64_t ldd, int bf16, cudaStream_t st);
cudaError_t launch_cast_rows64(const double* src, int64_t lds, int64_t rows, int cols, const float* rscale,
                               uint16_t* hi, uint16_t* lo, int64_t ldd, int bf16, cudaStream_t st);
cudaError_t launch_unscale_rows(float* X, int64_t ldx, int64_t rows, int cols, const float* rscale, cudaStream_t st);
// W: jacobi_w_doubles(l) (l x svd_bj_cols(l) for the block Jacobi), V: l x l, flags: >= 64 ints
cudaError_t launch_jacobi_svd(const float* R, int64_t ldr, int l, int r, double* W, double* V, double* sig, int* flags,
                              float* S, float* Ub, float* Vb, cudaStream_t st);
size_t jacobi_w_doubles(int l);
// ---- svd.cu (block one-sided Jacobi: 64-column block pairs on thread-block clusters)
bool svd_bj_fits(int l);
int svd_bj_cols(int l);
cudaError_t launch_svd_bj(double* W, int l, int max_sweeps, double tol, unsigned long long* maxoff, int* sweeps_out,
                          cudaStream_t st);

// ---- blas.cu (CGLS vectors, triangular inverse, small products)
// y = A x (fp32 A, fp64 x, y); with sq: also sq[sq_idx] = |y|^2 via sq_part (>= 1184 doubles)
cudaError_t launch_gemv_n(const float* A, int64_t lda, int64_t m, int n, const double* x, double* y, double* work,
                          const double* done, cudaStream_t st, double* sq = nullptr, int sq_idx = 0,
                          double* sq_part = nullptr);
size_t gemv_n_work_doubles(int64_t m, int n);
cudaError_t launch_gemv_t(const float* A, int64_t lda, int64_t m, int n, const double* r, double* s, double* work,
                          const double* done, cudaStream_t st);
size_t gemv_t_work_doubles(int64_t m, int n);
// one-pass q = A t, w = A^T q (CGLS, NEXT-4); sc[1] = |q|^2
size_t gemv_nt_work_doubles(int n);
bool gemv_nt_ok(const float* A, int64_t lda, int n);
cudaError_t launch_gemv_nt(const float* A, int64_t lda, int64_t m, int n, const double* t, double* q, double* w,
                           double* work, double* sc, cudaStream_t st);
cudaError_t launch_cgls_sv(double* sv, const double* w, int n, const double* sc, cudaStream_t st);
// Rinv: 2 n^2 doubles -- R^{-1} column-major, then its row-major copy (read by launch_trmv(.., 0, ..))
cudaError_t launch_trinv_upper(const float* R, int64_t ldr, int n, double* Rinv, cudaStream_t st);
cudaError_t launch_trmv(const double* Rinv, int n, const double* x, double* y, int transpose, const double* done,
                        cudaStream_t st);
cudaError_t launch_cgls_init(const float* b, int64_t m, int n, double* r, double* x, cudaStream_t st);
cudaError_t launch_sqnorm(const double* v, int64_t len, double* sc, int idx, cudaStream_t st);
cudaError_t launch_cgls_xr(double* x, const double* t, double* r, const double* q, int64_t m, int n, double* sc,
                           cudaStream_t st);
cudaError_t launch_cgls_p(const double* s, double* p, int n, double* sc, int first, cudaStream_t st);
// LSQR (right-preconditioned by R, same passes as CGLS): u = q - (alpha / beta) u, sc[1] = |u|^2
cudaError_t launch_lsqr_u(double* u, const double* q, int64_t m, double* sc, double* sqp, cudaStream_t st);
cudaError_t launch_lsqr_sv(double* sv, const double* w, int n, const double* sc, cudaStream_t st);
cudaError_t launch_lsqr_step(const double* p, double* v, double* w, double* y, int n, double* sc, int first,
                             cudaStream_t st);
cudaError_t launch_gaussian_philox(int64_t total, uint64_t seed, double* out64, float* out32, cudaStream_t st);
cudaError_t launch_philox_words(int64_t ncalls, uint64_t seed, uint32_t* words, cudaStream_t st);
size_t probe_work_doubles(int64_t m, int n, int p);
cudaError_t launch_orth_probe_z(const float* Q, int64_t ldq, int64_t m, int n, const double* G, double* work,
                                double* Z, cudaStream_t st);
cudaError_t launch_orth_probe_finish(const double* Z, int n, const double* G, double* out, cudaStream_t st);
cudaError_t launch_trmm_upper(const float* A, int64_t lda, const float* B, int64_t ldb, float* C, int64_t ldc, int n,
                              cudaStream_t st);

template <typename... KArgs, typename... Args>
inline cudaError_t launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                            Args&&... args) {
    ++g_launches;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl_enabled() ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

}  // namespace rg

