// panel_cholqr.cu -- CholQR2 leaf panel with an fp64 Gram matrix (north_star: "a
// bandwidth-bound panel MGS/CholQR kernel"; SURVEY 2.2 A19 / 8(e) "CholQR2 (fp64 Gram)").
//
//   pass 0:  G1 = P^T P                                   (fp64 accumulation)
//            -> R1 = chol(G1), R1^{-1}                    (last CTA, one warp)
//   pass 1:  Q1 = P R1^{-1} (fp32, registers only), G2 = Q1^T Q1
//            -> R2 = chol(G2), R2^{-1}
//   pass 2:  Q = (P R1^{-1}) R2^{-1}  -> Q (fp32) + 16-bit shadow;  R = R2 R1
//
// Q1 is recomputed in pass 2 with the same arithmetic as in pass 1 (bit-identical), so it
// is never stored: three reads of the panel (L2-resident at these sizes) and one write.
// Why this is the default B200 leaf: the MGS tiles of Alg 2 need 32
// dependent block-wide reductions per tile plus a tree of stacked-R factorisations, which
// is latency-bound on B200 (~240 us per 65536 x 32 panel measured); CholQR2 streams.
// With an fp64 Gram, Q1's orthogonality is ~kappa u32 and the second pass brings it to
// ~u32 while kappa(P) < ~1e7.  A failed pivot sets a device flag: the TSQR/MGS kernels of
// panel.cu (guarded by it) then redo the panel from the untouched input.
//
// Reductions are deterministic: CTA partials are summed in fixed order by the last CTA of
// each group of 16 ("last block" pattern), then by the last group.
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>

#include <algorithm>
#include <cstdlib>

#include <cooperative_groups.h>

#include "kernels.h"
#include "ptx.cuh"

namespace cg = cooperative_groups;

namespace rg {

constexpr int CQ_NB = 32;
constexpr int CQ_TILE = 128;          // rows staged per iteration
constexpr int CQ_LD = CQ_TILE + 4;    // smem column stride: 16-byte aligned columns; the DMMA
                                      // fragment reads (lane 4 g + c -> 4 g + c mod 32) stay conflict-free
constexpr int CQ_THREADS = 256;
constexpr int CQ_STAGES = 3;                        // cp.async ring depth of the streaming passes
constexpr int CQ_TILE_FLOATS = 32 * (CQ_TILE + 4);  // one 128 x 32 tile (column stride CQ_LD)
constexpr int CQ_FAN = 16;            // CTAs per reduction group

__device__ __forceinline__ uint16_t cq_to16(float x, int bf16) {
    if (bf16) {
        __nv_bfloat16 b = __float2bfloat16_rn(x);
        return *reinterpret_cast<uint16_t*>(&b);
    }
    __half h = __float2half_rn(x);
    return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float cq_from16(uint16_t u, int bf16) {
    if (bf16) return __bfloat162float(*reinterpret_cast<__nv_bfloat16*>(&u));
    return __half2float(*reinterpret_cast<__half*>(&u));
}

struct CqWs {            // device workspace layout (doubles unless noted)
    double* part;        // [grid][1024] CTA partial Grams
    double* gpart;       // [ngroups][1024] group partial Grams
    double* G;           // [2][1024] reduced Grams (distributed mode reads / writes these)
    double* R;           // [2][1024] Cholesky factors R1, R2 (fp64, upper, R[i + 32 j])
    float* Rinv;         // [2][1024] fp32 inverses R1^{-1}, R2^{-1}
    int* counters;       // [ngroups + 1], zero-initialised, self-resetting
    int* fail;           // 1 when a Cholesky pivot failed (guards the MGS fallback)
};

struct CqArgs {
    const float* P;      // panel (fp32, ldp); also the in-place output location
    int64_t ldp;
    float* Q;            // final Q, ldq (may alias P)
    int64_t ldq;
    uint16_t* Qh;        // 16-bit shadow (hi) of Q, ldh
    uint16_t* Ql;        // lo part (split mode) or null
    int64_t ldh;
    int64_t m;
    int nc;
    CqWs ws;
    float* Rout;         // final nc x nc R block (ldr)
    int64_t ldr;
    int bf16;
    int distributed;     // 1: stop after the reduced Gram; the host allreduces + factors
    unsigned long long cond;   // graph conditional handle of the MGS/TSQR fallback node (0: none)
    int* status;         // fused kernels: atomicMin(status, col0 + j) on a numerical breakdown
    int col0;            // global index of the panel's first column
    // fused kernels: Algorithm 1 line 9 for this panel first, P <- P - Q1 R12 (uh > 0)
    const float* uq;     // Q1 (fp32, m x uh, ld uq_ld)
    int64_t uq_ld;
    const float* ur;     // R12 (fp32, uh x nc, ld ur_ld)
    int64_t ur_ld;
    int uh;
};

// A failed pivot: raise the fallback flag and, inside a CUDA graph, switch on the conditional
// node that holds the MGS/TSQR kernels (so they are not launched at all on the common path).
__device__ __forceinline__ void cq_signal_fail(const CqArgs& a) {
    *a.ws.fail = 1;
    if (a.cond) cudaGraphSetConditional((cudaGraphConditionalHandle)a.cond, 1u);
}

// ---------------------------------------------------------------- Gram accumulation
// Streaming passes, on the fp64 tensor cores (DMMA m8n8k4): warp w takes the 4-row
// k-steps w, w + 8, ... of the 128-row tile and accumulates all 10 upper 8x8 blocks of the 32x32
// Gram (block t: (bi, bj) row by row); fragment b of a k-step is P[k0 + c][8 b + g] (lane = 4 g +
// c), converted once and used as both the A (P_bi^T) and B (P_bj) operand.  Replaces 4x4 DFMA
// blocks fed by 8 LDS + 8 F2F per 16 DFMA, which stalled on shared-memory latency (ncu:
// short_scoreboard, 12 % of DRAM peak).
__host__ __device__ constexpr int cq_blk_i(int t) { return t < 4 ? 0 : t < 7 ? 1 : t < 9 ? 2 : 3; }
__host__ __device__ constexpr int cq_blk_j(int t) { return t < 4 ? t : t < 7 ? t - 3 : t < 9 ? t - 5 : 3; }
template <int T>
__device__ __forceinline__ void cq_dmma(double (&acc)[10][2], const double (&f)[4]) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(acc[T][0]), "+d"(acc[T][1])
                 : "d"(f[cq_blk_i(T)]), "d"(f[cq_blk_j(T)]));
}
__device__ __forceinline__ void gram_dmma_accum(const float* tile, int rows, int warp, int lane, double (&acc)[10][2]) {
    const int g = lane >> 2, c = lane & 3;
    const float* col = tile + g * CQ_LD + c;
#pragma unroll 2
    for (int k0 = 4 * warp; k0 < rows; k0 += 32) {   // rows beyond `rows` in the last k-step are zero
        double f[4];
#pragma unroll
        for (int b = 0; b < 4; ++b) f[b] = (double)col[8 * b * CQ_LD + k0];
        cq_dmma<0>(acc, f); cq_dmma<1>(acc, f); cq_dmma<2>(acc, f); cq_dmma<3>(acc, f); cq_dmma<4>(acc, f);
        cq_dmma<5>(acc, f); cq_dmma<6>(acc, f); cq_dmma<7>(acc, f); cq_dmma<8>(acc, f); cq_dmma<9>(acc, f);
    }
}

// ---------------------------------------------------------------- Cholesky + inverse
// Whole CTA (blockDim.x == NT threads), N x N fp64 (N = 32 or 64), blocked by 4 columns:
// N / 4 block steps of
//   phase 1 (N / 32 warps): every lane factors the 4x4 diagonal block A_bb = L_bb L_bb^T in
//            registers (the only serial chain: 4 rsqrt), then lane l either forms one panel row
//            L_ib = A_ib L_bb^{-T} or applies L_bb^{-1} to one column of Z's block row b;
//   phase 2 (all warps): trailing update A_ij -= L_ib L_jb^T (i >= j) and Z_i -= L_ib Z_b,
// one barrier after each phase.  Z starts as I and ends as L^{-1} (the same block row operations
// applied to the identity), so one sweep yields R = L^T and R^{-1} = L^{-T}.  (A one-warp
// column-at-a-time version was ~8.5K straight-line SASS instructions and cost 35 us per panel
// cold; a one-barrier-per-column CTA version ~20K cycles.)
//   G     : upper triangle of the Gram, G[a + N b] (a <= b), nc x nc used; global or smem.
//   A, Z  : smem scratch, N x (N + 2) doubles each, 16-byte aligned; Z may alias G (G is read
//           completely before Z is initialised).  On exit A[i * (N + 2) + j] = R(i, j) (zero
//           below the diagonal).
//   Rg    : optional fp64 R, column-major [i + N j].
//   Rinvg : fp32 R^{-1}; row-major [i * N + j] if rinv_rowmajor else column-major [i + N j].
// Returns false (on every thread) if a pivot is not safely positive relative to G's diagonal
// (first such column in *first_bad, N if none); the factor is then garbage but finite.
constexpr int CH_LD = 34;   // N + 2 for N = 32: 16-byte aligned rows for the double2 loads
template <int NT, bool kSharedG, int N = 32>
__device__ bool chol_inv_cta(const double* G, int nc, double* A, double* Z, double* Rg, float* Rinvg,
                             bool rinv_rowmajor, int* first_bad = nullptr) {
    constexpr int LD = N + 2;
    static_assert(NT % 32 == 0 && (N * N) % NT == 0 && NT >= N, "thread count");
    constexpr int PER = N * N / NT;   // elements per thread (rows w + RS c, column tid % N)
    constexpr int RS = NT / N;        // row stride between a thread's elements
    __shared__ double odiag[N];
    __shared__ int s_bad;
    const int tid = threadIdx.x, lane = tid % N, rbase = tid / N;
    auto gload = [&](int a, int b) -> double { return kSharedG ? G[a + N * b] : __ldcg(G + a + N * b); };
#pragma unroll 4
    for (int c = 0; c < PER; ++c) {
        const int i = rbase + RS * c, j = lane;
        const double g = (i < nc && j < nc) ? gload(min(i, j), max(i, j)) : (i == j ? 1.0 : 0.0);
        A[i * LD + j] = g;
        if (i == j) odiag[i] = g;
    }
    if (tid == 0) s_bad = N;
    __syncthreads();
#pragma unroll 4
    for (int c = 0; c < PER; ++c) {
        const int i = rbase + RS * c, j = lane;
        Z[i * LD + j] = (i == j) ? 1.0 : 0.0;
    }
    __syncthreads();
#pragma unroll 1
    for (int k0 = 0; k0 < N; k0 += 4) {
        if (tid < N) {   // phase 1
            const int l = tid;
            const double* Ab = A + k0 * LD + k0;
            const double d00 = Ab[0];
            const double d10 = Ab[LD], d11 = Ab[LD + 1];
            const double d20 = Ab[2 * LD], d21 = Ab[2 * LD + 1], d22 = Ab[2 * LD + 2];
            const double d30 = Ab[3 * LD], d31 = Ab[3 * LD + 1], d32 = Ab[3 * LD + 2], d33 = Ab[3 * LD + 3];
            const int npan = N - 4 - k0;          // lanes < npan: panel row; others: Z column
            const bool pan = l < npan;
            const int r = k0 + 4 + l, col = l - npan;
            double p[4];
            if (pan) {
                const double2 v0 = *reinterpret_cast<const double2*>(A + r * LD + k0);
                const double2 v1 = *reinterpret_cast<const double2*>(A + r * LD + k0 + 2);
                p[0] = v0.x; p[1] = v0.y; p[2] = v1.x; p[3] = v1.y;
            } else {
#pragma unroll
                for (int c = 0; c < 4; ++c) p[c] = Z[(k0 + c) * LD + col];
            }
            if (N == 32) __syncwarp(); else asm volatile("bar.sync 1, %0;" :: "r"(N));   // all read A_bb
            int bad = N;
            auto piv = [&](double d, int kk) -> double {
                const bool gd = (d > odiag[kk] * 1e-15) && isfinite(d);
                if (!gd) bad = min(bad, kk);
                const double y = rsqrt(fmax(d, 1e-300));   // no branch on gd in the pivot chain
                return gd ? y : 1.0;
            };
            const double i0 = piv(d00, k0);
            const double l10 = d10 * i0, l20 = d20 * i0, l30 = d30 * i0;
            const double e11 = fma(-l10, l10, d11);
            const double i1 = piv(e11, k0 + 1);
            const double l21 = fma(-l20, l10, d21) * i1, l31 = fma(-l30, l10, d31) * i1;
            const double e22 = fma(-l21, l21, fma(-l20, l20, d22));
            const double i2 = piv(e22, k0 + 2);
            const double l32 = fma(-l31, l21, fma(-l30, l20, d32)) * i2;
            const double e33 = fma(-l32, l32, fma(-l31, l31, fma(-l30, l30, d33)));
            const double i3 = piv(e33, k0 + 3);
            const double m10 = -l10 * i0 * i1;
            const double m21 = -l21 * i1 * i2;
            const double m20 = -fma(l21, m10, l20 * i0) * i2;
            const double m32 = -l32 * i2 * i3;
            const double m31 = -fma(l32, m21, l31 * i1) * i3;
            const double m30 = -fma(l32, m20, fma(l31, m10, l30 * i0)) * i3;
            double q[4];
            q[0] = p[0] * i0;
            q[1] = fma(p[0], m10, p[1] * i1);
            q[2] = fma(p[0], m20, fma(p[1], m21, p[2] * i2));
            q[3] = fma(p[0], m30, fma(p[1], m31, fma(p[2], m32, p[3] * i3)));
            if (pan) {   // row r of L_ib = A_ib L_bb^{-T}
                *reinterpret_cast<double2*>(A + r * LD + k0) = make_double2(q[0], q[1]);
                *reinterpret_cast<double2*>(A + r * LD + k0 + 2) = make_double2(q[2], q[3]);
            } else {     // column col of Z_b <- L_bb^{-1} Z_b
#pragma unroll
                for (int c = 0; c < 4; ++c) Z[(k0 + c) * LD + col] = q[c];
            }
            if (l == 0) {
                double* Lb = A + k0 * LD + k0;   // L_bb (lower) in place of A_bb
                Lb[0] = d00 * i0;
                Lb[LD] = l10;
                Lb[LD + 1] = e11 * i1;
                Lb[2 * LD] = l20;
                Lb[2 * LD + 1] = l21;
                Lb[2 * LD + 2] = e22 * i2;
                Lb[3 * LD] = l30;
                Lb[3 * LD + 1] = l31;
                Lb[3 * LD + 2] = l32;
                Lb[3 * LD + 3] = e33 * i3;
                if (bad < s_bad) s_bad = bad;
            }
        }
        __syncthreads();
        // phase 2: rows i >= k0 + 4 (warp-uniform), column j = lane; operands loaded 4 rows at a
        // time before any store so the rows overlap instead of serialising on possible aliasing
        {
            const int j = lane;
            const bool zl = j < k0 + 4;   // Z column (else A column j)
            double ob[4];
            if (zl) {
#pragma unroll
                for (int c = 0; c < 4; ++c) ob[c] = Z[(k0 + c) * LD + j];
            } else {
                const double2 b0 = *reinterpret_cast<const double2*>(A + j * LD + k0);
                const double2 b1 = *reinterpret_cast<const double2*>(A + j * LD + k0 + 2);
                ob[0] = b0.x; ob[1] = b0.y; ob[2] = b1.x; ob[3] = b1.y;
            }
            const int cstart = (k0 + 4 - rbase + RS - 1) / RS;   // first c with row >= k0 + 4
#pragma unroll 1
            for (int c0 = cstart < 0 ? 0 : cstart; c0 < PER; c0 += 4) {
                double la[4][4], cur[4];
#pragma unroll
                for (int cc = 0; cc < 4; ++cc) {
                    const int i = rbase + RS * (c0 + cc);
                    if (c0 + cc < PER) {
                        const double2 a0 = *reinterpret_cast<const double2*>(A + i * LD + k0);
                        const double2 a1 = *reinterpret_cast<const double2*>(A + i * LD + k0 + 2);
                        la[cc][0] = a0.x; la[cc][1] = a0.y; la[cc][2] = a1.x; la[cc][3] = a1.y;
                        cur[cc] = zl ? Z[i * LD + j] : A[i * LD + j];
                    }
                }
#pragma unroll
                for (int cc = 0; cc < 4; ++cc) {
                    const int i = rbase + RS * (c0 + cc);
                    if (c0 + cc < PER) {
                        double v = cur[cc];
                        v = fma(-la[cc][0], ob[0], v);
                        v = fma(-la[cc][1], ob[1], v);
                        v = fma(-la[cc][2], ob[2], v);
                        v = fma(-la[cc][3], ob[3], v);
                        if (zl)
                            Z[i * LD + j] = v;
                        else if (j <= i)
                            A[i * LD + j] = v;
                    }
                }
            }
        }
        __syncthreads();
    }
    // outputs: R(i, j) = L(j, i), R^{-1}(i, j) = L^{-1}(j, i)
    const int nbad = s_bad;
    if (first_bad) *first_bad = nbad;
#pragma unroll 4
    for (int c = 0; c < PER; ++c) {
        const int i = rbase + RS * c, j = lane;
        const float ri = (i <= j) ? (float)Z[j * LD + i] : 0.f;
        Rinvg[rinv_rowmajor ? (i * N + j) : (i + N * j)] = ri;
        if (Rg) Rg[i + N * j] = (i <= j) ? A[j * LD + i] : 0.0;
    }
    __syncthreads();
    // A <- R row-major (upper): transpose the lower triangle in place, then clear it
#pragma unroll 4
    for (int c = 0; c < PER; ++c) {
        const int i = rbase + RS * c, j = lane;
        if (i < j) A[i * LD + j] = A[j * LD + i];
    }
    __syncthreads();
#pragma unroll 4
    for (int c = 0; c < PER; ++c) {
        const int i = rbase + RS * c, j = lane;
        if (i > j) A[i * LD + j] = 0.0;
    }
    __syncthreads();
    return nbad == N;
}

// Sum `n` partial Grams [n][1024] (upper triangle) in fixed order into dst (whole CTA);
// loads are issued CQ_FAN at a time before the adds so the latency is paid once per chunk.
__device__ void sum_parts(const double* src, int n, double* dst) {
    for (int e = threadIdx.x; e < 1024; e += blockDim.x) {
        const int i = e & 31, j = e >> 5;
        double s = 0.0;
        for (int c0 = 0; c0 < n; c0 += CQ_FAN) {
            double v[CQ_FAN];
#pragma unroll
            for (int c = 0; c < CQ_FAN; ++c)
                v[c] = (i <= j && c0 + c < n) ? __ldcg(src + (int64_t)(c0 + c) * 1024 + e) : 0.0;
#pragma unroll
            for (int c = 0; c < CQ_FAN; ++c) s += v[c];
        }
        dst[e] = s;
    }
}

// R = R2 R1 (fp64 product of upper-triangular factors; positive diagonal) -> a.Rout.
// R2 is in smem (Rs[i * CH_LD + j], left there by chol_inv_cta), R1 in the workspace.
__device__ void final_r_product(const CqArgs& a, const double* Rs, double* R1s /*smem 32x33*/) {
    for (int e = threadIdx.x; e < 1024; e += blockDim.x) R1s[(e & 31) * 33 + (e >> 5)] = __ldcg(a.ws.R + e);
    __syncthreads();
    for (int e = threadIdx.x; e < a.nc * a.nc; e += blockDim.x) {
        const int i = e % a.nc, j = e / a.nc;
        double s = 0.0;
        for (int k = i; k <= j; ++k) s = fma(Rs[i * CH_LD + k], R1s[k * 33 + j], s);
        a.Rout[i + (int64_t)j * a.ldr] = (i <= j) ? (float)s : 0.f;
    }
}

// kappa_F(R1) = |R1|_F |R1^{-1}|_F <= 2 nc  ->  one CholQR pass is enough (ws.fail[1] = 1).
__device__ void single_pass_decision(const CqArgs& a) {
    __shared__ double red[2][32];
    double r = 0.0, ri = 0.0;
    for (int e = threadIdx.x; e < 1024; e += blockDim.x) {
        const int i = e & 31, j = e >> 5;
        if (i < a.nc && j < a.nc) {
            const double x = __ldcg(a.ws.R + e);
            const double y = (double)__ldcg(a.ws.Rinv + e);
            r = fma(x, x, r);
            ri = fma(y, y, ri);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        r += __shfl_xor_sync(0xffffffffu, r, o);
        ri += __shfl_xor_sync(0xffffffffu, ri, o);
    }
    if ((threadIdx.x & 31) == 0) {
        red[0][threadIdx.x >> 5] = r;
        red[1][threadIdx.x >> 5] = ri;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double sr = 0.0, sri = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
            sr += red[0][w];
            sri += red[1][w];
        }
        a.ws.fail[1] = (sqrt(sr * sri) <= 2.0 * a.nc) ? 1 : 0;
    }
}

// Hierarchical last-block reduction + (single GPU) Cholesky of the reduced Gram.
__device__ void reduce_and_factor(const CqArgs& a, int pass, double* smem_R, double* smem_R1) {
    __shared__ int s_last;
    const int grid = gridDim.x;
    const int ngroups = (grid + CQ_FAN - 1) / CQ_FAN;
    const int grp = blockIdx.x / CQ_FAN;
    const int gsize = min(CQ_FAN, grid - grp * CQ_FAN);
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = (atomicAdd(&a.ws.counters[grp], 1) == gsize - 1);
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    sum_parts(a.ws.part + (int64_t)grp * CQ_FAN * 1024, gsize, a.ws.gpart + (int64_t)grp * 1024);
    if (threadIdx.x == 0) a.ws.counters[grp] = 0;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = (atomicAdd(&a.ws.counters[ngroups], 1) == ngroups - 1);
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    double* G = a.ws.G + pass * 1024;
    sum_parts(a.ws.gpart, ngroups, G);
    if (threadIdx.x == 0) a.ws.counters[ngroups] = 0;
    __threadfence();
    __syncthreads();
    if (a.distributed) return;   // host: allreduce(G) then cq_factor_kernel
    // smem_R1 doubles as the elimination scratch Y; final_r_product reloads it afterwards
    const bool ok = chol_inv_cta<CQ_THREADS, false>(G, a.nc, smem_R, smem_R1, a.ws.R + pass * 1024,
                                                     a.ws.Rinv + pass * 1024, false);
    if (!ok && threadIdx.x == 0) cq_signal_fail(a);
    if (pass == 0 && ok) single_pass_decision(a);
    if (pass == 1 && ok) final_r_product(a, smem_R, smem_R1);
}

// ---------------------------------------------------------------- streaming passes
// PASS 0: partial Gram of P -> (last CTA) R1, R1^{-1}, and the decision whether one
//         CholQR pass suffices (kappa_F(R1) = |R1|_F |R1^{-1}|_F <= 2 nc: Q1 = P R1^{-1} is
//         then orthogonal to a few u32, like one MGS pass), stored in ws.fail[1].
// PASS 1: Q1 = P R1^{-1}; single-pass panels write Q1 as Q (+ shadow) and R = R1;
//         otherwise partial Gram of Q1 -> (last CTA) R2, R2^{-1}, R = R2 R1.
// PASS 2: (two-pass panels only) Q = (P R1^{-1}) R2^{-1} (+ shadow).
//
// Per 128-row tile, thread t owns rows {t/8 + 32 i} (i < 4) and columns 4 (t%8) .. +3, so
// every shared-memory load of R^{-1} (one float4) feeds 16 FMAs.
__device__ __forceinline__ void tile_times_rinv(float* tile, const float* Rinv /*32 x 32, ld 32*/, int tid) {
    // thread (cgp = tid % 8, rq = tid / 8): rows 4 rq .. 4 rq + 3 (one float4 of the column) x
    // columns 4 cgp .. + 3: two 16-byte shared loads per 16 FMAs
    const int cgp = tid & 7, rq = tid >> 3;
    float o[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int c = 0; c < 4; ++c) o[i][c] = 0.f;
#pragma unroll 8
    for (int k = 0; k < CQ_NB; ++k) {
        const float4 rv = *reinterpret_cast<const float4*>(Rinv + k * 32 + 4 * cgp);
        const float4 xv = *reinterpret_cast<const float4*>(tile + k * CQ_LD + 4 * rq);
        const float x[4] = {xv.x, xv.y, xv.z, xv.w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            o[i][0] = fmaf(x[i], rv.x, o[i][0]);
            o[i][1] = fmaf(x[i], rv.y, o[i][1]);
            o[i][2] = fmaf(x[i], rv.z, o[i][2]);
            o[i][3] = fmaf(x[i], rv.w, o[i][3]);
        }
    }
    __syncthreads();
#pragma unroll
    for (int c = 0; c < 4; ++c)
        *reinterpret_cast<float4*>(tile + (4 * cgp + c) * CQ_LD + 4 * rq) =
            make_float4(o[0][c], o[1][c], o[2][c], o[3][c]);
    __syncthreads();
}

template <int PASS>
__global__ void __launch_bounds__(CQ_THREADS, 2) cq_pass_kernel(CqArgs a) {
    RG_PDL_ENTRY();
    __shared__ __align__(16) float tile_static[CQ_NB * CQ_LD + 64];   // also R1 scratch (32 x 33 doubles)
    extern __shared__ __align__(16) float ring[];                       // [CQ_STAGES][CQ_TILE_FLOATS]
    __shared__ __align__(16) float Ri[2][32 * 32];
    __shared__ __align__(16) double sred[2][1024];   // CTA partial-sum scratch (2 row groups at a time); reused
                                       // as the 32 x 33 Cholesky scratch by the last CTA
    const int tid = threadIdx.x;
    if (PASS == 0 && blockIdx.x == 0 && tid == 0) {
        a.ws.fail[0] = 0;
        a.ws.fail[1] = 0;
    }
    bool single = false;
    if (PASS > 0) {
        if (*(volatile int*)a.ws.fail) return;   // the MGS fallback owns this panel
        single = *(volatile int*)(a.ws.fail + 1) != 0;
        if (PASS == 2 && single) return;         // finished in pass 1
        for (int e = tid; e < 1024; e += CQ_THREADS) {
            Ri[0][e] = a.ws.Rinv[(e & 31) * 32 + (e >> 5)];   // Ri[k][j] = R^{-1}(k, j)
            if (PASS == 2) Ri[1][e] = a.ws.Rinv[1024 + (e & 31) * 32 + (e >> 5)];
        }
        if (PASS == 1 && single && blockIdx.x == 0)
            for (int e = tid; e < a.nc * a.nc; e += CQ_THREADS) {
                const int i = e % a.nc, j = e / a.nc;
                a.Rout[i + (int64_t)j * a.ldr] = (i <= j) ? (float)a.ws.R[i + 32 * j] : 0.f;
            }
    }
    const bool write_q = (PASS == 2) || (PASS == 1 && single);
    // 16-byte Q / 8-byte image stores need aligned column starts (rows per CTA and tiles are
    // multiples of 4)
    const bool vec = ((a.ldq & 3) == 0) && ((reinterpret_cast<uintptr_t>(a.Q) & 15) == 0) && ((a.ldh & 3) == 0) &&
                     ((reinterpret_cast<uintptr_t>(a.Qh) & 7) == 0) && ((reinterpret_cast<uintptr_t>(a.Ql) & 7) == 0);
    const bool gram = (PASS == 0) || (PASS == 1 && !single);
    const int warp = tid >> 5, lane = tid & 31;
    double acc[10][2] = {};
    const int64_t rows_per_cta = ((a.m + gridDim.x - 1) / gridDim.x + 3) / 4 * 4;
    const int64_t r0 = (int64_t)blockIdx.x * rows_per_cta;
    const int64_t r1 = min(a.m, r0 + rows_per_cta);
    // Tiles of 128 rows x 32 columns.  Aligned panels: a CQ_STAGES-deep cp.async ring in dynamic
    // shared memory (48 KB of loads in flight per CTA); otherwise a one-tile register prefetch.
    const bool async_ld = ((a.ldp & 3) == 0) && ((reinterpret_cast<uintptr_t>(a.P) & 15) == 0);
    auto issue = [&](int64_t tb, float* dst) {   // rows [tb, tb + 128) of the panel, 16-byte copies
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const int e = tid + k * CQ_THREADS;
            const int rq = e & 31, c = e >> 5;
            const int64_t gr = tb + 4 * rq;
            const int avail = (c < a.nc && gr < r1) ? (int)(r1 - gr < 4 ? r1 - gr : 4) : 0;
            const float* src = avail > 0 ? a.P + gr + (int64_t)c * a.ldp : a.P;
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst + c * CQ_LD + 4 * rq)),
                         "l"(src), "r"(avail * 4)
                         : "memory");
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    float pre[16];
    if (async_ld) {
#pragma unroll
        for (int sidx = 0; sidx < CQ_STAGES - 1; ++sidx) issue(r0 + (int64_t)sidx * CQ_TILE, ring + sidx * CQ_TILE_FLOATS);
    } else {
#pragma unroll
        for (int k = 0; k < 16; ++k) {
            const int e = tid + k * CQ_THREADS;
            const int r = e % CQ_TILE, c = e / CQ_TILE;
            pre[k] = (r0 + r < r1 && c < a.nc) ? a.P[r0 + r + (int64_t)c * a.ldp] : 0.f;
        }
    }
    int it = 0;
    for (int64_t base = r0; base < r1; base += CQ_TILE, ++it) {
        const int rows = (int)((r1 - base) < CQ_TILE ? (r1 - base) : CQ_TILE);
        float* tile = tile_static;
        if (async_ld) {
            issue(base + (int64_t)(CQ_STAGES - 1) * CQ_TILE, ring + ((it + CQ_STAGES - 1) % CQ_STAGES) * CQ_TILE_FLOATS);
            asm volatile("cp.async.wait_group %0;" ::"n"(CQ_STAGES - 1) : "memory");
            __syncthreads();
            tile = ring + (it % CQ_STAGES) * CQ_TILE_FLOATS;
        } else {
            __syncthreads();
#pragma unroll
            for (int k = 0; k < 16; ++k) {
                const int e = tid + k * CQ_THREADS;
                tile[(e / CQ_TILE) * CQ_LD + (e % CQ_TILE)] = pre[k];
            }
            __syncthreads();
            const int64_t nb = base + CQ_TILE;
#pragma unroll
            for (int k = 0; k < 16; ++k) {
                const int e = tid + k * CQ_THREADS;
                const int r = e % CQ_TILE, c = e / CQ_TILE;
                pre[k] = (nb + r < r1 && c < a.nc) ? a.P[nb + r + (int64_t)c * a.ldp] : 0.f;
            }
        }
        if (PASS > 0) {
            tile_times_rinv(tile, Ri[0], tid);                 // tile <- Q1 = P R1^{-1}
            if (PASS == 2) tile_times_rinv(tile, Ri[1], tid);  // tile <- Q = Q1 R2^{-1}
            if (write_q && vec) {
                // 4 consecutive rows of a column per thread: float4 Q, 8-byte 16-bit images
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const int e = tid + k * CQ_THREADS;
                    const int rq = e & 31, c = e >> 5;
                    const int r = 4 * rq;
                    if (c < a.nc && r < rows) {
                        const float4 v = *reinterpret_cast<const float4*>(tile + c * CQ_LD + r);
                        const int64_t gr = base + r;
                        if (r + 3 < rows) {
                            __stcs(reinterpret_cast<float4*>(a.Q + gr + (int64_t)c * a.ldq), v);
                            if (a.Qh) {   // packed (two-wide) conversions
                                uint2 hb, lb;
                                float2 h01, h23;
                                if (a.bf16) {
                                    const __nv_bfloat162 b01 = __floats2bfloat162_rn(v.x, v.y), b23 = __floats2bfloat162_rn(v.z, v.w);
                                    hb.x = *reinterpret_cast<const uint32_t*>(&b01);
                                    hb.y = *reinterpret_cast<const uint32_t*>(&b23);
                                    h01 = __bfloat1622float2(b01);
                                    h23 = __bfloat1622float2(b23);
                                } else {
                                    const __half2 b01 = __floats2half2_rn(v.x, v.y), b23 = __floats2half2_rn(v.z, v.w);
                                    hb.x = *reinterpret_cast<const uint32_t*>(&b01);
                                    hb.y = *reinterpret_cast<const uint32_t*>(&b23);
                                    h01 = __half22float2(b01);
                                    h23 = __half22float2(b23);
                                }
                                *reinterpret_cast<uint2*>(a.Qh + gr + (int64_t)c * a.ldh) = hb;
                                if (a.Ql) {
                                    const float l0 = (v.x - h01.x) * 2048.f, l1 = (v.y - h01.y) * 2048.f;
                                    const float l2 = (v.z - h23.x) * 2048.f, l3 = (v.w - h23.y) * 2048.f;
                                    if (a.bf16) {
                                        const __nv_bfloat162 c01 = __floats2bfloat162_rn(l0, l1), c23 = __floats2bfloat162_rn(l2, l3);
                                        lb.x = *reinterpret_cast<const uint32_t*>(&c01);
                                        lb.y = *reinterpret_cast<const uint32_t*>(&c23);
                                    } else {
                                        const __half2 c01 = __floats2half2_rn(l0, l1), c23 = __floats2half2_rn(l2, l3);
                                        lb.x = *reinterpret_cast<const uint32_t*>(&c01);
                                        lb.y = *reinterpret_cast<const uint32_t*>(&c23);
                                    }
                                    *reinterpret_cast<uint2*>(a.Ql + gr + (int64_t)c * a.ldh) = lb;
                                }
                            }
                        } else {
                            const float vv[4] = {v.x, v.y, v.z, v.w};
                            for (int u = 0; u < 4 && r + u < rows; ++u) {
                                a.Q[gr + u + (int64_t)c * a.ldq] = vv[u];
                                if (a.Qh) {
                                    const uint16_t hb = cq_to16(vv[u], a.bf16);
                                    a.Qh[gr + u + (int64_t)c * a.ldh] = hb;
                                    if (a.Ql)
                                        a.Ql[gr + u + (int64_t)c * a.ldh] =
                                            cq_to16((vv[u] - cq_from16(hb, a.bf16)) * 2048.f, a.bf16);
                                }
                            }
                        }
                    }
                }
            } else if (write_q) {
#pragma unroll
                for (int k = 0; k < 16; ++k) {
                    const int e = tid + k * CQ_THREADS;
                    const int r = e % CQ_TILE, c = e / CQ_TILE;
                    if (r < rows && c < a.nc) {
                        const float v = tile[c * CQ_LD + r];
                        const int64_t gr = base + r;
                        a.Q[gr + (int64_t)c * a.ldq] = v;
                        if (a.Qh) {
                            const uint16_t hb = cq_to16(v, a.bf16);
                            a.Qh[gr + (int64_t)c * a.ldh] = hb;
                            if (a.Ql) a.Ql[gr + (int64_t)c * a.ldh] = cq_to16((v - cq_from16(hb, a.bf16)) * 2048.f,
                                                                               a.bf16);
                        }
                    }
                }
            }
        }
        if (gram) gram_dmma_accum(tile, rows, warp, lane, acc);
        if (async_ld) __syncthreads();   // this ring slot is refilled by the next iteration
    }
    if (!gram) return;
    // ---- CTA partial Gram: the 8 warps' block accumulators summed in warp order (2 warps at a
    // time through smem: slot (w & 1) * 640 + block * 64 + 2 lane + v)
    double* out = a.ws.part + (int64_t)blockIdx.x * 1024;
    double* sw = &sred[0][0];
    double run[4] = {0.0, 0.0, 0.0, 0.0};
    for (int round = 0; round < 4; ++round) {
        __syncthreads();
        if ((warp >> 1) == round) {
#pragma unroll
            for (int t = 0; t < 10; ++t) {
                sw[(warp & 1) * 640 + t * 64 + 2 * lane] = acc[t][0];
                sw[(warp & 1) * 640 + t * 64 + 2 * lane + 1] = acc[t][1];
            }
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int e = tid + CQ_THREADS * q;
            const int i = e & 31, j = e >> 5;
            if (i <= j) {
                const int bi = i >> 3, bj = j >> 3;
                const int t = bi == 0 ? bj : bi == 1 ? 3 + bj : bi == 2 ? 5 + bj : 9;
                const int idx = t * 64 + 2 * (4 * (i & 7) + ((j & 7) >> 1)) + (j & 1);
                run[q] += sw[idx];
                run[q] += sw[640 + idx];
            }
        }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int e = tid + CQ_THREADS * q;
        const int i = e & 31, j = e >> 5;
        out[e] = (i <= j) ? run[q] : 0.0;
    }
    __syncthreads();
    reduce_and_factor(a, PASS, &sred[0][0], reinterpret_cast<double*>(tile_static));
}


// ---------------------------------------------------------------- fused single-kernel panel
// Whole CholQR2 panel of NC = 32 or 64 columns in one cooperative kernel (rows per CTA must fit
// in shared memory): every CTA keeps its rows of the panel in shared memory for the whole
// computation, so the panel is read once and written once; the Gram reductions run through a
// fixed-order last-arriver tree + flag broadcast (cf_allreduce) and every CTA factors the reduced
// Gram itself (identical arithmetic on identical data -> identical R on every CTA).
//
// NC = 64 covers the last recursion level of Algorithm 1 with two 32-column panels at once:
// with G = [P1 P2]^T [P1 P2], the recursion step computes R11 = chol(G11), R12 = Q1^T P2 =
// R11^{-T} G12 and R22 = chol(G22 - R12^T R12), which is the Cholesky factor of the 64 x 64 G;
// so in exact arithmetic the 64-column CholQR2 returns the same (unique) Q and R as the two
// panels + K1 + K2 of that level, and the second CholQR pass restores orthogonality exactly as
// it does for a 32-column panel.
constexpr int CF_THREADS = 256;
constexpr int CF_FAN = 8;                        // CTA partials per first-level group
constexpr int CF_MAX_ROWS = 1280;                // rows per CTA that fit next to the scratch (NC = 32)
constexpr int CF_WIDE_MAX_ROWS = 560;            // same for NC = 64
constexpr int CF_MAXPER = CF_MAX_ROWS / CF_THREADS;   // tile rows per thread (load / store loops)
constexpr int CF_NE_MAX = 64 * 65 / 2;           // packed Gram entries, NC = 64

template <int NC>
struct CfCfg {
    static constexpr int NE = NC * (NC + 1) / 2;             // packed upper-triangle entries
};

__device__ __forceinline__ void tri_unpack(int p, int& i, int& j) {
    int jj = (int)((sqrtf(8.f * p + 1.f) - 1.f) * 0.5f);
    if ((jj + 1) * (jj + 2) / 2 <= p) ++jj;
    if (jj * (jj + 1) / 2 > p) --jj;
    j = jj;
    i = p - jj * (jj + 1) / 2;
}

// Gram partial of the CTA's tile rows [0, rows) (NC columns) -> out (fp64, packed upper
// triangle [j (j + 1) / 2 + i]) on the fp64 tensor cores (mma.sync m8n8k4 f64: 256 FMAs per
// warp instruction).  Rows are converted to fp64 once per chunk into a row-major staging
// buffer (row stride SLD = NC + 4 == 4 mod 16 doubles: the 4 rows x 8 columns of a fragment hit
// distinct banks).  Warp w takes the 4-row k-steps w, w + 8, ... and keeps one accumulator per
// 8x8 block of the upper triangle, so its DMMAs are independent and the NB8 fragments it loads
// per k-step are reused by every block (A and B of a Gram are the same rows).  The eight warp
// partials are then added in warp order through the scratch (fixed order: deterministic).
template <int NC>
__device__ void cf_gram(const float* tile, int ld, int rows, double* S, int s_cap, double* out_partial) {
    constexpr int NB8 = NC / 8, NBLK = NB8 * (NB8 + 1) / 2, SLD = NC + 4;
    constexpr int NW = CF_THREADS / 32;
    const int CH = s_cap / SLD / 32 * 32;                 // rows per chunk, whole k-step rounds
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int g = lane >> 2, c = lane & 3;
    double acc[NBLK][2];
#pragma unroll
    for (int t = 0; t < NBLK; ++t) acc[t][0] = acc[t][1] = 0.0;
    for (int ch0 = 0; ch0 < rows; ch0 += CH) {
        const int cr = min(CH, rows - ch0), cr4 = (cr + 3) & ~3;
        __syncthreads();
        // fp32 -> fp64 staging, 8 conversions in flight per thread
        for (int e0 = 0; e0 < cr4 * NC; e0 += 8 * CF_THREADS) {
            float x[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const int e = e0 + tid + u * CF_THREADS, r = e / NC, col = e % NC;
                x[u] = (r < cr) ? tile[col * ld + ch0 + r] : 0.f;
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const int e = e0 + tid + u * CF_THREADS, r = e / NC, col = e % NC;
                if (e < cr4 * NC) S[r * SLD + col] = (double)x[u];
            }
        }
        __syncthreads();
        for (int k0 = 4 * warp; k0 < cr4; k0 += 4 * NW) {
            const double* rowp = S + (k0 + c) * SLD + g;
            double f[NB8];
#pragma unroll
            for (int bi = 0; bi < NB8; ++bi) f[bi] = rowp[bi * 8];
            int t = 0;
#pragma unroll
            for (int bi = 0; bi < NB8; ++bi)
#pragma unroll
                for (int bj = bi; bj < NB8; ++bj, ++t)
                    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                                 : "+d"(acc[t][0]), "+d"(acc[t][1])
                                 : "d"(f[bi]), "d"(f[bj]));
        }
    }
    // warp partials -> S in rounds of WPR warps, summed in warp order by all threads; entry
    // e = (t * 2 + u) * 32 + lane (block t, element u of this lane's D fragment)
    constexpr int NENT = NBLK * 64;
    const int WPR = s_cap / NENT < NW ? s_cap / NENT : NW;
    constexpr int NQ = (NENT + CF_THREADS - 1) / CF_THREADS;
    double run[NQ];
#pragma unroll
    for (int q = 0; q < NQ; ++q) run[q] = 0.0;
    for (int w0 = 0; w0 < NW; w0 += WPR) {
        __syncthreads();
        if (warp >= w0 && warp < w0 + WPR) {
            double* dst = S + (warp - w0) * NENT + lane;
#pragma unroll
            for (int t = 0; t < NBLK; ++t) {
                dst[(t * 2 + 0) * 32] = acc[t][0];
                dst[(t * 2 + 1) * 32] = acc[t][1];
            }
        }
        __syncthreads();
        const int nw = min(WPR, NW - w0);
#pragma unroll
        for (int q = 0; q < NQ; ++q) {
            const int e = tid + CF_THREADS * q;
            if (e < NENT)
                for (int k = 0; k < nw; ++k) run[q] += S[k * NENT + e];
        }
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < NQ; ++q) {
        const int e = tid + CF_THREADS * q;
        if (e < NENT) S[e] = run[q];
    }
    __syncthreads();
    // D fragment of block (bi, bj): lane holds rows g, columns 2c, 2c + 1
    for (int e = tid; e < CfCfg<NC>::NE; e += CF_THREADS) {
        int i, j;
        tri_unpack(e, i, j);
        const int bi = i >> 3, bj = j >> 3;
        const int t = bi * NB8 - bi * (bi - 1) / 2 + (bj - bi);
        const int ln = (i & 7) * 4 + ((j & 7) >> 1), u = j & 1;
        out_partial[e] = S[(t * 2 + u) * 32 + ln];
    }
    __syncthreads();
}

#ifdef RG_CF_TRACE
__device__ unsigned long long cf_trace[16];
#define CF_MARK(i)                                                                     \
    do {                                                                               \
        if (blockIdx.x == 0 && threadIdx.x == 0) {                                     \
            unsigned long long t;                                                      \
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));                      \
            cf_trace[i] = t;                                                           \
        }                                                                              \
    } while (0)
#else
#define CF_MARK(i) \
    do {           \
    } while (0)
#endif

// Counter slots used by the fused kernels (the streaming passes use [0, ngroups]): one 128-byte
// line each, so the 147 CTAs polling the flag do not queue behind the arrival atomics.
constexpr int CF_CNT_BASE = 1024, CF_CNT_STRIDE = 32;
constexpr int CF_CNT_GLOBAL = CF_CNT_BASE + 20 * CF_CNT_STRIDE, CF_CNT_FLAG = CF_CNT_BASE + 21 * CF_CNT_STRIDE;
constexpr int CF_CNT_INTS = CF_CNT_BASE + 22 * CF_CNT_STRIDE;

__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Workspace of the fused kernels (doubles): CTA partials [160][NE], group sums [20][NE],
// reduced Gram [NE], accumulated R [NC * NC] (CTA 0 only).
struct CfWs {
    double* part;
    double* gpart;
    double* G;
    double* Racc;
};
__device__ __forceinline__ CfWs cf_ws(const CqArgs& a) {
    CfWs w;
    w.part = a.ws.part;
    w.gpart = w.part + (size_t)160 * CF_NE_MAX;
    w.G = w.gpart + (size_t)20 * CF_NE_MAX;
    w.Racc = w.G + CF_NE_MAX;
    return w;
}
constexpr size_t CF_WS_DOUBLES = (size_t)(160 + 20 + 1) * CF_NE_MAX + 64 * 64;

// Grid-wide fixed-order reduction of the CTA partials (NE doubles each) into Gs (smem, fp64,
// [i + NC j]) on every CTA, without grid barriers: the last CTA to arrive in each group of
// CF_FAN sums the group's partials, the last group to finish sums the group sums into w.G and
// bumps a generation flag; every CTA spins on the flag and reads the NE entries.  Every sum has
// a fixed order (CTA order within a group, group order), so the result is bitwise reproducible.
template <int NC>
__device__ void cf_allreduce(const CqArgs& a, double* Gs) {
    constexpr int NE = CfCfg<NC>::NE;
    constexpr int NQ = (NE + CF_THREADS - 1) / CF_THREADS;      // entries per thread
    constexpr int MAXG = (160 + CF_FAN - 1) / CF_FAN;           // grid <= 160 CTAs
    const CfWs w = cf_ws(a);
    const int ngroups = (gridDim.x + CF_FAN - 1) / CF_FAN;
    const int grp = blockIdx.x / CF_FAN;
    const int gsize = min(CF_FAN, (int)gridDim.x - grp * CF_FAN);
    const int tid = threadIdx.x;
    int* cnt = a.ws.counters;
    unsigned* flag = reinterpret_cast<unsigned*>(cnt + CF_CNT_FLAG);
    int* gcnt = cnt + CF_CNT_BASE + grp * CF_CNT_STRIDE;
    __shared__ int s_last;
    __shared__ unsigned s_gen;
    if (tid == 0) s_gen = *(volatile unsigned*)flag;   // read before this CTA arrives
    fence_acq_rel_gpu();
    __syncthreads();
    if (tid == 0) s_last = (atomicAdd(gcnt, 1) == gsize - 1);
    __syncthreads();
    if (s_last) {
        fence_acq_rel_gpu();
        const int c0 = grp * CF_FAN;
#pragma unroll 3
        for (int q = 0; q < NQ; ++q) {
            const int e = tid + CF_THREADS * q;
            double v[CF_FAN];
#pragma unroll
            for (int c = 0; c < CF_FAN; ++c)
                v[c] = (c < gsize && e < NE) ? __ldcg(w.part + (int64_t)(c0 + c) * NE + e) : 0.0;
            double sum = 0.0;
#pragma unroll
            for (int c = 0; c < CF_FAN; ++c) sum += v[c];
            if (e < NE) w.gpart[(int64_t)grp * NE + e] = sum;
        }
        if (tid == 0) *gcnt = 0;
        fence_acq_rel_gpu();
        __syncthreads();
        if (tid == 0) s_last = (atomicAdd(cnt + CF_CNT_GLOBAL, 1) == ngroups - 1);
        __syncthreads();
        if (s_last) {
            fence_acq_rel_gpu();
#pragma unroll 1
            for (int q = 0; q < NQ; ++q) {
                const int e = tid + CF_THREADS * q;
                if (e < NE) {
                    double v[MAXG];
#pragma unroll
                    for (int g = 0; g < MAXG; ++g) v[g] = (g < ngroups) ? __ldcg(w.gpart + (int64_t)g * NE + e) : 0.0;
                    double sum = 0.0;
#pragma unroll
                    for (int g = 0; g < MAXG; ++g) sum += v[g];
                    w.G[e] = sum;
                }
            }
            if (tid == 0) cnt[CF_CNT_GLOBAL] = 0;
            fence_acq_rel_gpu();
            __syncthreads();
            if (tid == 0) atomicAdd(flag, 1u);
        }
    }
    if (tid == 0)
        while (ld_acquire_gpu(flag) == s_gen) __nanosleep(100);
    __syncthreads();
    fence_acq_rel_gpu();
    {   // all of this thread's loads in flight before the unpack/stores (one L2 round trip)
        constexpr int MQ = (NE + CF_THREADS - 1) / CF_THREADS;
        double v[MQ];
#pragma unroll
        for (int u = 0; u < MQ; ++u) {
            const int e = tid + u * CF_THREADS;
            v[u] = e < NE ? __ldcg(w.G + e) : 0.0;
        }
#pragma unroll
        for (int u = 0; u < MQ; ++u) {
            const int e = tid + u * CF_THREADS;
            if (e < NE) {
                int i, j;
                tri_unpack(e, i, j);
                Gs[i + NC * j] = v[u];
            }
        }
    }
    __syncthreads();
}

// tile (rows x NC, ld) <- tile * Rinv (NC x NC fp32, row-major [k * NC + j]); each thread owns 4
// rows x 4 columns of a chunk, so every float4 of R^{-1} feeds 16 FMAs.
template <int NC>
__device__ void cf_times_rinv(float* tile, int ld, int rows, const float* Rinv) {
    constexpr int CG = NC / 4, RG = CF_THREADS / CG;   // column groups of 4 x row groups
    const int tid = threadIdx.x;
    const int cgp = tid % CG, rgp = tid / CG;
    for (int base = 0; base < rows; base += 4 * RG) {
        float o[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int c = 0; c < 4; ++c) o[i][c] = 0.f;
#pragma unroll 8
        for (int k = 0; k < NC; ++k) {
            const float4 rv = *reinterpret_cast<const float4*>(Rinv + k * NC + 4 * cgp);
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int r = base + rgp + RG * i;
                const float x = (r < rows) ? tile[k * ld + r] : 0.f;
                o[i][0] = fmaf(x, rv.x, o[i][0]);
                o[i][1] = fmaf(x, rv.y, o[i][1]);
                o[i][2] = fmaf(x, rv.z, o[i][2]);
                o[i][3] = fmaf(x, rv.w, o[i][3]);
            }
        }
        __syncthreads();
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int r = base + rgp + RG * i;
            if (r < rows)
#pragma unroll
                for (int c = 0; c < 4; ++c) tile[(4 * cgp + c) * ld + r] = o[i][c];
        }
        __syncthreads();
    }
}

// Shared memory of the fused kernels beyond the row tile: Gs, then Rs, Ri and all remaining
// shared memory, which the Gram staging S reuses (S is dead between the Gram of a pass and the
// elimination of the next; Rs / Ri are dead between the R^{-1} product and the next Gram).
template <int NC>
struct CfBufs {
    double* Gs;    // NC x (NC + 2): reduced Gram [i + NC j]; the elimination's Z aliases it
    double* Rs;    // NC x (NC + 2): elimination A; R of the last pass (row-major) on exit
    float* Ri;     // NC x NC fp32 R^{-1} of the last pass, row-major
    double* S;     // fp64 staging / warp partials of the Gram (aliases Rs, Ri, ...)
    int s_cap;     // doubles available at S
    static constexpr size_t fixed_bytes = (size_t)(2 * NC * (NC + 2)) * 8 + (size_t)NC * NC * 4;
    __device__ CfBufs(uint8_t* base, int cap) {
        Gs = reinterpret_cast<double*>(base);
        Rs = Gs + NC * (NC + 2);
        Ri = reinterpret_cast<float*>(Rs + NC * (NC + 2));
        S = Rs;
        s_cap = cap;
    }
};

// CholQR2 of the CTA's rows of one <= NC-column panel (tile, zero-padded to NC columns), all
// CTAs in lockstep through cf_allreduce.  Pass 1 forms G = P^T P (fp64), R1 = chol(G),
// Q1 = P R1^{-1}; kappa_F(R1) = |R1|_F |R1^{-1}|_F <= 2 nc ends the panel after one pass,
// otherwise pass 2 repeats it on Q1 (CholQR2).  If a pivot of pass 1 fails, the pass is redone
// on G + s I with the shifted-CholQR shift s = 11 (m nc + nc (nc + 1)) u ||P||_F^2 (u = 2^-53)
// and two more passes follow (shifted CholQR3), all inside the kernel.  A pivot that fails after
// that is a numerical breakdown: its column is reported through a.status and returned (else -1).
// On exit the tile holds Q and CTA 0 has written R (fp32) to a.Rout.
template <int NC>
__device__ int cf_panel(const CqArgs& a, float* tile, int ld, int rows, int nc, const CfBufs<NC>& b) {
    const int tid = threadIdx.x;
    const CfWs w = cf_ws(a);
    __shared__ int s_single;
    double* part = w.part + (int64_t)blockIdx.x * CfCfg<NC>::NE;
    bool shifted = false;
    int bad = -1;
    for (int pass = 0; pass < 3; ++pass) {
        cf_gram<NC>(tile, ld, rows, b.S, b.s_cap, part);
        CF_MARK(4 + 4 * pass);
        cf_allreduce<NC>(a, b.Gs);
        CF_MARK(5 + 4 * pass);
        int fb = NC;
        bool ok = chol_inv_cta<CF_THREADS, true, NC>(b.Gs, nc, b.Rs, b.Gs, nullptr, b.Ri, true, &fb);
        CF_MARK(6 + 4 * pass);
        if (!ok && pass == 0) {
            // reload G (the elimination overwrote it) and shift its diagonal
            for (int e = tid; e < CfCfg<NC>::NE; e += CF_THREADS) {
                int i, j;
                tri_unpack(e, i, j);
                b.Gs[i + NC * j] = __ldcg(w.G + e);
            }
            __syncthreads();
            double tr = 0.0;
            for (int j = 0; j < nc; ++j) tr += b.Gs[j * (NC + 1)];
            const double sh = 11.0 * ((double)a.m * nc + (double)nc * (nc + 1)) * 0x1p-53 * tr;
            __syncthreads();
            if (tid < nc) b.Gs[tid * (NC + 1)] += sh;
            __syncthreads();
            shifted = true;
            ok = chol_inv_cta<CF_THREADS, true, NC>(b.Gs, nc, b.Rs, b.Gs, nullptr, b.Ri, true, &fb);
        }
        if (!ok) {
            bad = fb;
            break;
        }
        // CTA 0 accumulates R = R_pass ... R_1 (fp64, [i + NC j]) in the workspace
        if (blockIdx.x == 0) {
            constexpr int PERQ = NC * NC / CF_THREADS;
            double v[PERQ];
#pragma unroll
            for (int q = 0; q < PERQ; ++q) {
                const int e = tid + CF_THREADS * q, i = e % NC, j = e / NC;
                double sacc = 0.0;
                if (i <= j) {
                    if (pass == 0) {
                        sacc = b.Rs[i * (NC + 2) + j];
                    } else {
                        for (int k = i; k <= j; ++k) sacc = fma(b.Rs[i * (NC + 2) + k], w.Racc[k + NC * j], sacc);
                    }
                }
                v[q] = sacc;
            }
            __syncthreads();
#pragma unroll
            for (int q = 0; q < PERQ; ++q) w.Racc[tid + CF_THREADS * q] = v[q];
        }
        bool stop;
        if (pass == 0) {
            if (tid < 32) {
                double r = 0.0, ri = 0.0;
                for (int e = tid; e < NC * NC; e += 32) {
                    const int i = e / NC, j = e % NC;
                    if (i < nc && j < nc) {
                        const double x = b.Rs[i * (NC + 2) + j];
                        const double y = (double)b.Ri[e];
                        r = fma(x, x, r);
                        ri = fma(y, y, ri);
                    }
                }
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    r += __shfl_xor_sync(0xffffffffu, r, o);
                    ri += __shfl_xor_sync(0xffffffffu, ri, o);
                }
                if (tid == 0) s_single = (sqrt(r * ri) <= 2.0 * nc) ? 1 : 0;
            }
            __syncthreads();
            stop = !shifted && s_single != 0;
        } else {
            __syncthreads();
            stop = (pass == 1 && !shifted) || pass == 2;
        }
        cf_times_rinv<NC>(tile, ld, rows, b.Ri);
        CF_MARK(7 + 4 * pass);
        if (stop) break;
    }
    if (bad >= 0 && blockIdx.x == 0 && tid == 0 && a.status) atomicMin(a.status, a.col0 + bad);
    if (blockIdx.x == 0) {   // R (fp32) from the accumulated fp64 factor (written by this CTA)
        __syncthreads();
        for (int e = tid; e < nc * nc; e += CF_THREADS) {
            const int i = e % nc, j = e / nc;
            a.Rout[i + (int64_t)j * a.ldr] = (i <= j) ? (float)w.Racc[i + NC * j] : 0.f;
        }
    }
    return bad;
}

// P <- P - Q1 R12 on the CTA's rows (Algorithm 1 line 9 for the panel that follows an update):
// the leaf-level K2 folded into the panel's load instead of a separate read-modify-write pass
// over the panel.  fp32 Q1 and R12 (the values the tensor-core K2 rounds to 16 bit), fp32 FMAs.
// R12 is staged in S as [k * NC + j]; Q1 in chunks of 128 rows as [k * 132 + r].
template <int NC>
__device__ void cf_pre_update(const CqArgs& a, float* tile, int ld, int rows, int64_t r0, double* Sd, int s_cap) {
    constexpr int CG = NC / 4, RG = CF_THREADS / CG;
    const int tid = threadIdx.x, cgp = tid % CG, rgp = tid / CG;
    const int uh = a.uh;
    float* Rf = reinterpret_cast<float*>(Sd);
    float* Qc = Rf + 64 * NC;
    // all of the CTA's Q1 rows at once when they fit (one round of loads), else 128-row chunks
    const int cap_rows = (int)(((int64_t)s_cap * 2 - 64 * NC) / (uh > 0 ? uh : 1)) - 4;
    const int chunk = rows <= cap_rows ? ((rows + 3) & ~3) : 4 * RG;
    const int qld = chunk + 4;
    for (int e = tid; e < uh * NC; e += CF_THREADS) {
        const int k = e / NC, j = e % NC;
        Rf[e] = (j < a.nc) ? a.ur[k + (int64_t)j * a.ur_ld] : 0.f;
    }
    for (int base = 0; base < rows; base += chunk) {
        const int cr = min(chunk, rows - base);
        __syncthreads();
        for (int e0 = 0; e0 < uh * cr; e0 += 8 * CF_THREADS) {
            float x[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const int e = e0 + tid + u * CF_THREADS, k = e / cr, r = e % cr;
                x[u] = (e < uh * cr) ? a.uq[r0 + base + r + (int64_t)k * a.uq_ld] : 0.f;
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const int e = e0 + tid + u * CF_THREADS, k = e / cr, r = e % cr;
                if (e < uh * cr) Qc[k * qld + r] = x[u];
            }
        }
        __syncthreads();
        for (int sb = 0; sb < cr; sb += 4 * RG) {
            float o[4][4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int r = sb + rgp + RG * i;
#pragma unroll
                for (int c = 0; c < 4; ++c) o[i][c] = (r < cr) ? tile[(4 * cgp + c) * ld + base + r] : 0.f;
            }
#pragma unroll 8
            for (int k = 0; k < uh; ++k) {
                const float4 rv = *reinterpret_cast<const float4*>(Rf + k * NC + 4 * cgp);
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const int r = sb + rgp + RG * i;
                    const float x = (r < cr) ? Qc[k * qld + r] : 0.f;
                    o[i][0] = fmaf(-x, rv.x, o[i][0]);
                    o[i][1] = fmaf(-x, rv.y, o[i][1]);
                    o[i][2] = fmaf(-x, rv.z, o[i][2]);
                    o[i][3] = fmaf(-x, rv.w, o[i][3]);
                }
            }
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int r = sb + rgp + RG * i;
                if (r < cr)
#pragma unroll
                    for (int c = 0; c < 4; ++c) tile[(4 * cgp + c) * ld + base + r] = o[i][c];
            }
        }
    }
    __syncthreads();
}

template <int NC>
__global__ void __launch_bounds__(CF_THREADS, 1) cq_fused_kernel(CqArgs a, int ld, int s_cap) {
    RG_PDL_ENTRY();
    extern __shared__ __align__(16) uint8_t cf_smem[];
    float* tile = reinterpret_cast<float*>(cf_smem);
    const CfBufs<NC> b(cf_smem + (((size_t)NC * ld * 4 + 15) & ~(size_t)15), s_cap);
    const int tid = threadIdx.x;
    if (blockIdx.x == 0 && tid == 0) *a.ws.fail = 0;
    const int64_t rows_per = (a.m + gridDim.x - 1) / gridDim.x;
    const int64_t r0 = (int64_t)blockIdx.x * rows_per;
    const int64_t rem = a.m - r0;
    const int rows = (int)(rem <= 0 ? 0 : (rem < rows_per ? rem : rows_per));
    CF_MARK(0);
    // ---- load the CTA's rows (zero-padded columns beyond nc); 4 columns x CF_MAXPER rows of
    // independent loads in flight per thread
    for (int c0 = 0; c0 < NC; c0 += 4) {
        float v[4][CF_MAXPER];
#pragma unroll
        for (int cc = 0; cc < 4; ++cc)
#pragma unroll
            for (int q = 0; q < CF_MAXPER; ++q) {
                const int r = tid + CF_THREADS * q, c = c0 + cc;
                v[cc][q] = (r < rows && c < a.nc) ? a.P[r0 + r + (int64_t)c * a.ldp] : 0.f;
            }
#pragma unroll
        for (int cc = 0; cc < 4; ++cc)
#pragma unroll
            for (int q = 0; q < CF_MAXPER; ++q) {
                const int r = tid + CF_THREADS * q;
                if (r < rows) tile[(c0 + cc) * ld + r] = v[cc][q];
            }
    }
    __syncthreads();
    if (a.uh > 0) cf_pre_update<NC>(a, tile, ld, rows, r0, b.S, b.s_cap);
    CF_MARK(1);
    cf_panel<NC>(a, tile, ld, rows, a.nc, b);
    CF_MARK(2);
    // ---- write Q (fp32) + 16-bit shadow
    for (int c = 0; c < a.nc; ++c) {
#pragma unroll
        for (int q = 0; q < CF_MAXPER; ++q) {
            const int r = tid + CF_THREADS * q;
            if (r < rows) {
                const float v = tile[c * ld + r];
                const int64_t gr = r0 + r;
                a.Q[gr + (int64_t)c * a.ldq] = v;
                if (a.Qh) {
                    const uint16_t hb = cq_to16(v, a.bf16);
                    a.Qh[gr + (int64_t)c * a.ldh] = hb;
                    if (a.Ql) a.Ql[gr + (int64_t)c * a.ldh] = cq_to16((v - cq_from16(hb, a.bf16)) * 2048.f, a.bf16);
                }
            }
        }
    }
    CF_MARK(3);
}

// distributed mode: after the host allreduce of G (pass `pass`), factor it (one warp)
__global__ void cq_factor_kernel(CqArgs a, int pass) {
    RG_PDL_ENTRY();
    __shared__ __align__(16) double Rs[32 * CH_LD];
    __shared__ __align__(16) double R1s[32 * CH_LD];
    // pass 1 runs only for two-pass panels: a single-pass panel (ws.fail[1], decided after pass
    // 0) has already written Q and R, and its second Gram was never formed (the host allreduce
    // of that slot is issued regardless and carries stale data)
    if (pass > 0 && (*(volatile int*)a.ws.fail || *(volatile int*)(a.ws.fail + 1))) return;
    const bool ok = chol_inv_cta<256, false>(a.ws.G + pass * 1024, a.nc, Rs, R1s, a.ws.R + pass * 1024,
                                             a.ws.Rinv + pass * 1024, false);
    if (!ok && threadIdx.x == 0) cq_signal_fail(a);
    if (pass == 0 && ok) single_pass_decision(a);
    if (pass == 1 && ok) final_r_product(a, Rs, R1s);
}

// ------------------------------------------------------------------ host side
static int cq_grid(int64_t m) {
    int64_t g = (m + 127) / 128;   // one or two 128-row tiles per CTA, two CTAs per SM
    if (g > 296) g = 296;
    if (g < 1) g = 1;
    return (int)g;
}

size_t cholqr_ws_doubles(int64_t m) {
    const int grid = cq_grid(m);
    const int ngroups = (grid + CQ_FAN - 1) / CQ_FAN;
    const size_t streaming = (size_t)(grid + ngroups) * 1024 + 4 * 1024 + 1024 /*Rinv fp32 x2*/ + 64;
    return std::max(streaming, CF_WS_DOUBLES + 64);   // the fused kernels' layout (cf_ws)
}

size_t cholqr_counter_ints(int64_t m) {
    const int grid = cq_grid(m);
    return std::max((size_t)(grid + CQ_FAN - 1) / CQ_FAN + 2, (size_t)CF_CNT_INTS);
}


static int sm_count() { return dev_sms(); }

bool cholqr_fused_fits(int64_t m, int ncols) {
    const int64_t rows_per = (m + sm_count() - 1) / sm_count();
    return rows_per <= (ncols > 32 ? CF_WIDE_MAX_ROWS : CF_MAX_ROWS) && getenv("RGSQR_CQ_STREAM") == nullptr;
}

static CqArgs cq_args(const CholqrLaunch& L) {
    CqArgs a{};
    a.P = L.P;
    a.ldp = L.ldp;
    a.Q = L.Q;
    a.ldq = L.ldq;
    a.Qh = L.Qh;
    a.Ql = L.Ql;
    a.ldh = L.ldh;
    a.m = L.m;
    a.nc = L.nc;
    const int grid = cq_grid(L.m);
    const int ngroups = (grid + CQ_FAN - 1) / CQ_FAN;
    a.ws.part = L.ws;
    a.ws.gpart = a.ws.part + (size_t)grid * 1024;
    a.ws.G = a.ws.gpart + (size_t)ngroups * 1024;
    a.ws.R = a.ws.G + 2048;
    a.ws.Rinv = reinterpret_cast<float*>(a.ws.R + 2048);
    a.ws.counters = L.counter;
    a.ws.fail = L.fail;
    a.Rout = L.R;
    a.ldr = L.ldr;
    a.bf16 = L.bf16;
    a.distributed = L.allreduce_g != nullptr;
    a.cond = L.cond;
    a.status = L.status;
    a.col0 = L.col0;
    a.uq = L.uq;
    a.uq_ld = L.uq_ld;
    a.ur = L.ur;
    a.ur_ld = L.ur_ld;
    a.uh = L.uh;
    return a;
}

template <int NC>
static cudaError_t launch_fused(CqArgs a, cudaStream_t st) {
    const int sms = sm_count();
    const int64_t rows_per = (a.m + sms - 1) / sms;
    const int ld = (int)(rows_per | 1);   // odd leading dimension: conflict-free column walks
    // all of shared memory: the tile, Gs, and the rest for Rs / Ri / Gram staging
    const int smem_max = dev_smem_optin() - 2048;   // static shared memory of the kernel + slack
    const size_t tile_bytes = (((size_t)NC * ld * 4 + 15) & ~(size_t)15);
    const size_t gs_bytes = (size_t)NC * (NC + 2) * 8;
    if (tile_bytes + CfBufs<NC>::fixed_bytes > (size_t)smem_max) return cudaErrorInvalidValue;
    const int s_cap = (int)(((size_t)smem_max - tile_bytes - gs_bytes) / 8);
    const size_t smem = (size_t)smem_max;
    cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(cq_fused_kernel<NC>), smem);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(sms);
    cfg.blockDim = dim3(CF_THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeCooperative;   // co-residency for the flag spin in cf_allreduce
    at[0].val.cooperative = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    ++g_launches;
    return cudaLaunchKernelEx(&cfg, cq_fused_kernel<NC>, a, ld, s_cap);
}

cudaError_t launch_panel_cholqr(const CholqrLaunch& L, bool* handles_failure, cudaStream_t st) {
    CqArgs a = cq_args(L);
    const int grid = cq_grid(L.m);
    if (L.uh > 0 && (a.distributed || !cholqr_fused_fits(L.m, 32) || L.uh > 64)) return cudaErrorInvalidValue;
    if (!a.distributed && cholqr_fused_fits(L.m, 32)) {
        if (handles_failure) *handles_failure = true;   // shifted CholQR3 inside the kernel
        return launch_fused<32>(a, st);
    }
    if (handles_failure) *handles_failure = false;      // the guarded MGS/TSQR kernels must follow
    cudaError_t e;
    constexpr size_t ring_bytes = (size_t)CQ_STAGES * CQ_TILE_FLOATS * 4;
    if ((e = ensure_smem_attr(reinterpret_cast<const void*>(cq_pass_kernel<0>), ring_bytes)) != cudaSuccess ||
        (e = ensure_smem_attr(reinterpret_cast<const void*>(cq_pass_kernel<1>), ring_bytes)) != cudaSuccess ||
        (e = ensure_smem_attr(reinterpret_cast<const void*>(cq_pass_kernel<2>), ring_bytes)) != cudaSuccess)
        return e;
    for (int pass = 0; pass < 3; ++pass) {
        if (pass == 0) RG_LAUNCH((cq_pass_kernel<0>), grid, CQ_THREADS, ring_bytes, st, a);
        if (pass == 1) RG_LAUNCH((cq_pass_kernel<1>), grid, CQ_THREADS, ring_bytes, st, a);
        if (pass == 2) RG_LAUNCH((cq_pass_kernel<2>), grid, CQ_THREADS, ring_bytes, st, a);
        e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        if (a.distributed && pass < 2) {
            if (L.allreduce_g(a.ws.G + pass * 1024, L.ctx) != 0) return cudaErrorUnknown;
            RG_LAUNCH((cq_factor_kernel), 1, 256, 0, st, a, pass);
            e = cudaGetLastError();
            if (e != cudaSuccess) return e;
        }
    }
    return cudaSuccess;
}

cudaError_t launch_panel_pair(const CholqrLaunch& L, cudaStream_t st) {
    if (L.nc <= 32 || L.nc > 64 || L.allreduce_g != nullptr || !cholqr_fused_fits(L.m, 64))
        return cudaErrorInvalidValue;
    return launch_fused<64>(cq_args(L), st);
}

}  // namespace rg
