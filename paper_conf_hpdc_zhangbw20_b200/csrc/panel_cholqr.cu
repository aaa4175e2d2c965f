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

namespace cg = cooperative_groups;

namespace rg {

constexpr int CQ_NB = 32;
constexpr int CQ_TILE = 128;          // rows staged per iteration
constexpr int CQ_LD = CQ_TILE + 1;    // smem column stride (bank-conflict-free column access)
constexpr int CQ_THREADS = 256;
constexpr int CQ_BLK = 36;            // 4x4 blocks in the upper triangle of a 32x32 Gram (8*9/2)
constexpr int CQ_GROUPS = CQ_THREADS / CQ_BLK;  // 7 row groups of 36 threads
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
};

// ---------------------------------------------------------------- Gram accumulation
__device__ __forceinline__ void blk_coords(int blk, int& bi, int& bj) {
    int b = 0, rem = blk;
    while (rem >= 8 - b) {
        rem -= 8 - b;
        ++b;
    }
    bi = b;
    bj = b + rem;
}

__device__ __forceinline__ void gram_block_accum(const float* tile, int rows, int g, int bi, int bj,
                                                 double (&acc)[4][4]) {
    for (int r = g; r < rows; r += CQ_GROUPS) {
        double x[4], y[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            x[u] = (double)tile[(bi * 4 + u) * CQ_LD + r];
            y[u] = (double)tile[(bj * 4 + u) * CQ_LD + r];
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int v = 0; v < 4; ++v) acc[u][v] = fma(x[u], y[v], acc[u][v]);
    }
}

// ---------------------------------------------------------------- Cholesky + inverse
// Whole CTA (blockDim.x == NT threads), 32 x 32 fp64, blocked by 4 columns: 8 block steps of
//   phase 1 (warp 0): every lane factors the 4x4 diagonal block A_bb = L_bb L_bb^T in registers
//            (the only serial chain: 4 rsqrt), then lane l either forms one panel row
//            L_ib = A_ib L_bb^{-T} or applies L_bb^{-1} to one column of Z's block row b;
//   phase 2 (all warps): trailing update A_ij -= L_ib L_jb^T (i >= j) and Z_i -= L_ib Z_b,
// one barrier after each phase.  Z starts as I and ends as L^{-1} (the same block row operations
// applied to the identity), so one sweep yields R = L^T and R^{-1} = L^{-T}.  (A one-warp
// column-at-a-time version was ~8.5K straight-line SASS instructions and cost 35 us per panel
// cold; a one-barrier-per-column CTA version ~20K cycles.)
//   G     : upper triangle of the Gram, G[a + 32 b] (a <= b), nc x nc used; global or smem.
//   A, Z  : smem scratch, 32 x CH_LD each, 16-byte aligned.  On exit A[i * CH_LD + j] = R(i, j)
//           (zero below the diagonal).
//   Rg    : optional fp64 R, column-major [i + 32 j].
//   Rinvg : fp32 R^{-1}; row-major [i * 32 + j] if rinv_rowmajor else column-major [i + 32 j].
// Returns false (on every thread) if a pivot is not safely positive relative to G's diagonal;
// the factor is then garbage but finite (pivot replaced by 1).
constexpr int CH_LD = 34;   // even: 16-byte aligned rows for the 2 x double2 panel loads
#ifdef RG_CHOL_TRACE
__device__ long long chol_trace[40];
__device__ long long chol_t0;
#endif
template <int NT, bool kSharedG>
__device__ bool chol_inv_cta(const double* G, int nc, double* A, double* Z, double* Rg, float* Rinvg,
                             bool rinv_rowmajor) {
    static_assert(NT % 32 == 0 && 1024 % NT == 0, "thread count");
    constexpr int PER = 1024 / NT;
    constexpr int NW = NT / 32;
    __shared__ double odiag[32];
    __shared__ int s_ok;
    const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
    auto gload = [&](int a, int b) -> double { return kSharedG ? G[a + 32 * b] : __ldcg(G + a + 32 * b); };
#pragma unroll
    for (int c = 0; c < PER; ++c) {
        const int e = tid + NT * c, i = e >> 5, j = e & 31;
        const double g = (i < nc && j < nc) ? gload(min(i, j), max(i, j)) : (i == j ? 1.0 : 0.0);
        A[i * CH_LD + j] = g;
        Z[i * CH_LD + j] = (i == j) ? 1.0 : 0.0;
        if (i == j) odiag[i] = g;
    }
    if (tid == 0) s_ok = 1;
    __syncthreads();
#pragma unroll 1
    for (int k0 = 0; k0 < 32; k0 += 4) {
#ifdef RG_CHOL_TRACE
        if (tid == 0) chol_trace[k0 / 4] = clock64();
#endif
        if (w == 0) {
            const double* Ab = A + k0 * CH_LD + k0;
            const double d00 = Ab[0];
            const double d10 = Ab[CH_LD], d11 = Ab[CH_LD + 1];
            const double d20 = Ab[2 * CH_LD], d21 = Ab[2 * CH_LD + 1], d22 = Ab[2 * CH_LD + 2];
            const double d30 = Ab[3 * CH_LD], d31 = Ab[3 * CH_LD + 1], d32 = Ab[3 * CH_LD + 2],
                         d33 = Ab[3 * CH_LD + 3];
            const int npan = 28 - k0;          // lanes < npan: panel row; others: Z column (npan + k0 + 4 = 32)
            const bool pan = lane < npan;
            const int r = k0 + 4 + lane, col = lane - npan;
            double p[4];
            if (pan) {
                const double2 v0 = *reinterpret_cast<const double2*>(A + r * CH_LD + k0);
                const double2 v1 = *reinterpret_cast<const double2*>(A + r * CH_LD + k0 + 2);
                p[0] = v0.x; p[1] = v0.y; p[2] = v1.x; p[3] = v1.y;
            } else {
#pragma unroll
                for (int c = 0; c < 4; ++c) p[c] = Z[(k0 + c) * CH_LD + col];
            }
            __syncwarp();   // every lane has read A_bb before lane 0 overwrites it with L_bb
            bool good = true;
            auto piv = [&](double d, int kk) -> double {
                const bool gd = (d > odiag[kk] * 1e-15) && isfinite(d);
                good = good && gd;
                const double y = rsqrt(fmax(d, 1e-300));   // no branch on gd in the pivot chain
                return gd ? y : 1.0;
            };
            const double i0 = piv(d00, k0);
            const double l10 = d10 * i0, l20 = d20 * i0, l30 = d30 * i0;
            const double i1 = piv(fma(-l10, l10, d11), k0 + 1);
            const double l21 = fma(-l20, l10, d21) * i1, l31 = fma(-l30, l10, d31) * i1;
            const double i2 = piv(fma(-l21, l21, fma(-l20, l20, d22)), k0 + 2);
            const double l32 = fma(-l31, l21, fma(-l30, l20, d32)) * i2;
            const double e33 = fma(-l32, l32, fma(-l31, l31, fma(-l30, l30, d33)));
            const double i3 = piv(e33, k0 + 3);
            // L_bb^{-1} (lower; diagonal i0..i3)
            const double m10 = -l10 * i0 * i1;
            const double m21 = -l21 * i1 * i2;
            const double m20 = -fma(l21, m10, l20 * i0) * i2;
            const double m32 = -l32 * i2 * i3;
            const double m31 = -fma(l32, m21, l31 * i1) * i3;
            const double m30 = -fma(l32, m20, fma(l31, m10, l30 * i0)) * i3;
            double q[4];
            if (pan) {   // row r of L_ib = A_ib L_bb^{-T}: q_c = sum_{k <= c} p_k Linv(c, k)
                q[0] = p[0] * i0;
                q[1] = fma(p[0], m10, p[1] * i1);
                q[2] = fma(p[0], m20, fma(p[1], m21, p[2] * i2));
                q[3] = fma(p[0], m30, fma(p[1], m31, fma(p[2], m32, p[3] * i3)));
                *reinterpret_cast<double2*>(A + r * CH_LD + k0) = make_double2(q[0], q[1]);
                *reinterpret_cast<double2*>(A + r * CH_LD + k0 + 2) = make_double2(q[2], q[3]);
            } else {     // column col of Z_b <- L_bb^{-1} Z_b (same formula)
                q[0] = p[0] * i0;
                q[1] = fma(m10, p[0], p[1] * i1);
                q[2] = fma(m20, p[0], fma(m21, p[1], p[2] * i2));
                q[3] = fma(m30, p[0], fma(m31, p[1], fma(m32, p[2], p[3] * i3)));
#pragma unroll
                for (int c = 0; c < 4; ++c) Z[(k0 + c) * CH_LD + col] = q[c];
            }
            if (lane == 0) {
                double* Lb = A + k0 * CH_LD + k0;   // L_bb (lower) in place of A_bb
                Lb[0] = d00 * i0;
                Lb[CH_LD] = l10;
                Lb[CH_LD + 1] = fma(-l10, l10, d11) * i1;
                Lb[2 * CH_LD] = l20;
                Lb[2 * CH_LD + 1] = l21;
                Lb[2 * CH_LD + 2] = fma(-l21, l21, fma(-l20, l20, d22)) * i2;
                Lb[3 * CH_LD] = l30;
                Lb[3 * CH_LD + 1] = l31;
                Lb[3 * CH_LD + 2] = l32;
                Lb[3 * CH_LD + 3] = e33 * i3;
                if (!good) s_ok = 0;
            }
#ifdef RG_CHOL_TRACE
            if (tid == 0) chol_trace[10 + k0 / 4] = clock64();
#endif
        }
        __syncthreads();
#ifdef RG_CHOL_TRACE
        if (tid == 0) chol_trace[20 + k0 / 4] = clock64();
#endif
        // phase 2: rows i >= k0 + 4 (warp-uniform), lane = column.  All operands are loaded
        // before any store so the PER rows overlap instead of serialising on possible aliasing.
        {
            const bool zl = lane < k0 + 4;   // Z column (else A column lane)
            double ob[4];
            if (zl) {
#pragma unroll
                for (int c = 0; c < 4; ++c) ob[c] = Z[(k0 + c) * CH_LD + lane];
            } else {
                const double2 b0 = *reinterpret_cast<const double2*>(A + lane * CH_LD + k0);
                const double2 b1 = *reinterpret_cast<const double2*>(A + lane * CH_LD + k0 + 2);
                ob[0] = b0.x; ob[1] = b0.y; ob[2] = b1.x; ob[3] = b1.y;
            }
            double la[PER][4], cur[PER];
#pragma unroll
            for (int c = 0; c < PER; ++c) {
                const int i = w + NW * c;
                if (i >= k0 + 4) {
                    const double2 a0 = *reinterpret_cast<const double2*>(A + i * CH_LD + k0);
                    const double2 a1 = *reinterpret_cast<const double2*>(A + i * CH_LD + k0 + 2);
                    la[c][0] = a0.x; la[c][1] = a0.y; la[c][2] = a1.x; la[c][3] = a1.y;
                    cur[c] = zl ? Z[i * CH_LD + lane] : A[i * CH_LD + lane];
                }
            }
#pragma unroll
            for (int c = 0; c < PER; ++c) {
                const int i = w + NW * c;
                if (i >= k0 + 4) {
                    double v = cur[c];
                    v = fma(-la[c][0], ob[0], v);
                    v = fma(-la[c][1], ob[1], v);
                    v = fma(-la[c][2], ob[2], v);
                    v = fma(-la[c][3], ob[3], v);
                    if (zl)
                        Z[i * CH_LD + lane] = v;
                    else if (lane <= i)
                        A[i * CH_LD + lane] = v;
                }
            }
        }
#ifdef RG_CHOL_TRACE
        if (tid == 0) chol_trace[30 + k0 / 4] = clock64();
#endif
        __syncthreads();
    }
#ifdef RG_CHOL_TRACE
    if (tid == 0) chol_trace[8] = clock64();
#endif
    double r[PER];
#pragma unroll
    for (int c = 0; c < PER; ++c) {
        const int e = tid + NT * c, i = e >> 5, j = e & 31;
        r[c] = (i <= j) ? A[j * CH_LD + i] : 0.0;                     // R(i, j) = L(j, i)
        const float ri = (i <= j) ? (float)Z[j * CH_LD + i] : 0.f;    // R^{-1}(i, j) = L^{-1}(j, i)
        Rinvg[rinv_rowmajor ? (i * 32 + j) : (i + 32 * j)] = ri;
        if (Rg) Rg[i + 32 * j] = r[c];
    }
    const bool ok = s_ok != 0;
    __syncthreads();
#pragma unroll
    for (int c = 0; c < PER; ++c) {
        const int e = tid + NT * c;
        A[(e >> 5) * CH_LD + (e & 31)] = r[c];
    }
    __syncthreads();
    return ok;
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
    if (!ok && threadIdx.x == 0) *a.ws.fail = 1;
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
    const int cgp = tid & 7, rgp = tid >> 3;
    float o[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int c = 0; c < 4; ++c) o[i][c] = 0.f;
#pragma unroll 8
    for (int k = 0; k < CQ_NB; ++k) {
        const float4 rv = *reinterpret_cast<const float4*>(Rinv + k * 32 + 4 * cgp);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const float x = tile[k * CQ_LD + rgp + 32 * i];
            o[i][0] = fmaf(x, rv.x, o[i][0]);
            o[i][1] = fmaf(x, rv.y, o[i][1]);
            o[i][2] = fmaf(x, rv.z, o[i][2]);
            o[i][3] = fmaf(x, rv.w, o[i][3]);
        }
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int c = 0; c < 4; ++c) tile[(4 * cgp + c) * CQ_LD + rgp + 32 * i] = o[i][c];
    __syncthreads();
}

template <int PASS>
__global__ void __launch_bounds__(CQ_THREADS, 2) cq_pass_kernel(CqArgs a) {
    RG_PDL_ENTRY();
    __shared__ __align__(16) float tile[CQ_NB * CQ_LD + 64];   // also R1 scratch (32 x 33 doubles)
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
    const bool gram = (PASS == 0) || (PASS == 1 && !single);
    const int g = tid / CQ_BLK, blk = tid % CQ_BLK;
    int bi, bj;
    blk_coords(blk, bi, bj);
    double acc[4][4] = {};
    const int64_t rows_per_cta = ((a.m + gridDim.x - 1) / gridDim.x + 3) / 4 * 4;
    const int64_t r0 = (int64_t)blockIdx.x * rows_per_cta;
    const int64_t r1 = min(a.m, r0 + rows_per_cta);
    // register prefetch of the next tile: thread loads element (r = e % 128, c = e / 128)
    float pre[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) {
        const int e = tid + k * CQ_THREADS;
        const int r = e % CQ_TILE, c = e / CQ_TILE;
        pre[k] = (r0 + r < r1 && c < a.nc) ? a.P[r0 + r + (int64_t)c * a.ldp] : 0.f;
    }
    for (int64_t base = r0; base < r1; base += CQ_TILE) {
        const int rows = (int)((r1 - base) < CQ_TILE ? (r1 - base) : CQ_TILE);
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
        if (PASS > 0) {
            tile_times_rinv(tile, Ri[0], tid);                 // tile <- Q1 = P R1^{-1}
            if (PASS == 2) tile_times_rinv(tile, Ri[1], tid);  // tile <- Q = Q1 R2^{-1}
            if (write_q) {
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
        if (gram && g < CQ_GROUPS) gram_block_accum(tile, rows, g, bi, bj, acc);
    }
    if (!gram) return;
    // ---- CTA partial Gram: sum the 7 row-group accumulators (2 at a time through smem)
    double* out = a.ws.part + (int64_t)blockIdx.x * 1024;
    for (int round = 0; round < 4; ++round) {
        const int g0 = round * 2;
        __syncthreads();
        for (int e = tid; e < 2 * 1024; e += CQ_THREADS) (&sred[0][0])[e] = 0.0;
        __syncthreads();
        if (g >= g0 && g < g0 + 2 && g < CQ_GROUPS) {
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int v = 0; v < 4; ++v) sred[g - g0][(bi * 4 + u) + (bj * 4 + v) * 32] = acc[u][v];
        }
        __syncthreads();
        for (int e = tid; e < 1024; e += CQ_THREADS) {
            const int i = e & 31, j = e >> 5;
            double s = (round == 0) ? 0.0 : out[e];
            s += sred[0][e] + sred[1][e];
            out[e] = (i <= j) ? s : 0.0;
        }
    }
    __syncthreads();
    reduce_and_factor(a, PASS, &sred[0][0], reinterpret_cast<double*>(tile));
}


// ---------------------------------------------------------------- fused single-kernel panel
// Whole CholQR2 panel in one cooperative kernel (m <= CF_MAX_ROWS * gridDim): every CTA keeps
// its rows of the panel in shared memory for the whole computation, so the panel is read once
// and written once; the three launches, two "last block" chains and the broadcast of R^{-1}
// of the streaming version become grid barriers, and every CTA factors the reduced 32 x 32
// Gram itself (identical arithmetic on identical data -> identical R on every CTA).
constexpr int CF_THREADS = 256;
constexpr int CF_GB = 10;                        // 8x8 blocks in the upper triangle of a 32x32 Gram (4*5/2)
constexpr int CF_GROUPS = CF_THREADS / CF_GB;    // 25 row groups of 10 threads (250 active)
constexpr int CF_CH = 96;                        // rows staged in fp64 per Gram chunk
constexpr int CF_SLD = 34;                       // fp64 row stride of the staging chunk (16B-aligned rows)
constexpr int CF_SCR = CF_CH * CF_SLD;           // scratch doubles: staging chunk / 5 group partials / Y
constexpr int CF_FAN = 8;                        // CTA partials per first-level group
constexpr int CF_MAX_ROWS = 1280;                // rows per CTA that fit next to the scratch
constexpr int CF_MAXPER = CF_MAX_ROWS / CF_THREADS;   // tile rows per thread (load / store loops)
static_assert(CF_GROUPS % 5 == 0 && 5 * 641 <= CF_SCR && 32 * CH_LD <= CF_SCR, "Gram scratch");

struct CfSmem {
    static size_t bytes(int ld) {
        return (size_t)32 * ld * 4        // tile (column-major, ld)
               + CF_SCR * 8               // fp64 staging / reduction / elimination scratch
               + 32 * CH_LD * 8 * 2       // G (padded) + Cholesky scratch
               + 2 * 32 * 32 * 4          // R1^{-1}, R2^{-1} (fp32, [k][j])
               + 1024 * 8                 // R1 (fp64) kept for R = R2 R1
               + 256;
    }
};

constexpr int CF_NP = 32 * 33 / 2;               // packed upper-triangle entries of a partial Gram
__device__ __forceinline__ void tri_unpack(int p, int& i, int& j) {
    int jj = (int)((sqrtf(8.f * p + 1.f) - 1.f) * 0.5f);
    if ((jj + 1) * (jj + 2) / 2 <= p) ++jj;
    if (jj * (jj + 1) / 2 > p) --jj;
    j = jj;
    i = p - jj * (jj + 1) / 2;
}

__device__ __forceinline__ void cf_blk_coords(int blk, int& bi, int& bj) {
    // (0,0) (0,1) (0,2) (0,3) (1,1) (1,2) (1,3) (2,2) (2,3) (3,3)
    bi = blk < 4 ? 0 : (blk < 7 ? 1 : (blk < 9 ? 2 : 3));
    bj = bi + blk - (bi == 0 ? 0 : (bi == 1 ? 4 : (bi == 2 ? 7 : 9)));
}

// Gram partial of the CTA's tile rows [0, rows) -> out (fp64, packed upper triangle
// [j (j + 1) / 2 + i], CF_NP entries), fixed order.  Rows are converted to fp64 once per CF_CH-row chunk (row-major staging,
// so each thread's 8 consecutive columns are 4 LDS.128), then 8x8 register blocks give 4 DFMA per
// loaded double: the loop runs at the fp64 FMA rate instead of the F2F conversion rate.
__device__ void cf_gram(const float* tile, int ld, int rows, double* S, double* out_partial) {
    const int tid = threadIdx.x;
    const int g = tid / CF_GB, blk = tid % CF_GB;
    int bi = 0, bj = 0;
    cf_blk_coords(blk, bi, bj);
    double acc[8][8];
#pragma unroll
    for (int u = 0; u < 8; ++u)
#pragma unroll
        for (int v = 0; v < 8; ++v) acc[u][v] = 0.0;
    for (int ch0 = 0; ch0 < rows; ch0 += CF_CH) {
        const int cr = min(CF_CH, rows - ch0);
        __syncthreads();
        for (int e = tid; e < cr * 32; e += CF_THREADS) {
            const int r = e >> 5, c = e & 31;
            S[r * CF_SLD + c] = (double)tile[c * ld + ch0 + r];
        }
        __syncthreads();
        if (g < CF_GROUPS) {
            for (int r = g; r < cr; r += CF_GROUPS) {
                const double2* row = reinterpret_cast<const double2*>(S + r * CF_SLD);
                double x[8], y[8];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const double2 vx = row[bi * 4 + q], vy = row[bj * 4 + q];
                    x[2 * q] = vx.x;
                    x[2 * q + 1] = vx.y;
                    y[2 * q] = vy.x;
                    y[2 * q + 1] = vy.y;
                }
#pragma unroll
                for (int u = 0; u < 8; ++u)
#pragma unroll
                    for (int v = 0; v < 8; ++v) acc[u][v] = fma(x[u], y[v], acc[u][v]);
            }
        }
    }
    // fixed-order sum of the 25 group accumulators, 5 groups per round through S
    // (entry e = (u * 8 + v) * 10 + blk, group stride 641: conflict-free stores and loads)
    double run[3] = {0.0, 0.0, 0.0};   // entries tid, tid + 256, tid + 512 (< 640)
    for (int round = 0; round < CF_GROUPS / 5; ++round) {
        __syncthreads();
        const int gl = g - 5 * round;
        if (g < CF_GROUPS && gl >= 0 && gl < 5) {
#pragma unroll
            for (int u = 0; u < 8; ++u)
#pragma unroll
                for (int v = 0; v < 8; ++v) S[gl * 641 + (u * 8 + v) * 10 + blk] = acc[u][v];
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 3; ++q) {
            const int e = tid + CF_THREADS * q;
            if (e < 640) run[q] += ((S[e] + S[641 + e]) + (S[1282 + e] + S[1923 + e])) + S[2564 + e];
        }
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < 3; ++q) {
        const int e = tid + CF_THREADS * q;
        if (e < 640) S[e] = run[q];
    }
    __syncthreads();
    for (int e = tid; e < CF_NP; e += CF_THREADS) {
        int i, j;
        tri_unpack(e, i, j);
        double v;
        {
            const int pi = i >> 3, pj = j >> 3;
            const int b = (pi == 0 ? 0 : (pi == 1 ? 4 : (pi == 2 ? 7 : 9))) + (pj - pi);
            v = S[((i & 7) * 8 + (j & 7)) * 10 + b];
        }
        out_partial[e] = v;
    }
    __syncthreads();
}

// Grid-wide fixed-order reduction of the CTA partials into Gs (smem, fp64, upper) on every CTA.
#ifdef RG_CF_TRACE
__device__ unsigned long long cf_trace[16];
__device__ unsigned long long cf_cta[4][160];
#define CF_CTA(i)                                                                      \
    do {                                                                               \
        if (threadIdx.x == 0) {                                                        \
            unsigned long long t;                                                      \
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));                      \
            cf_cta[i][blockIdx.x] = t;                                                 \
        }                                                                              \
    } while (0)
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
#define CF_CTA(i) \
    do {          \
    } while (0)
#endif

// Counter slots used by the fused kernel (the streaming passes use [0, ngroups]): one 128-byte
// line each, so the 147 CTAs polling the flag do not queue behind the arrival atomics.
constexpr int CF_CNT_BASE = 1024, CF_CNT_STRIDE = 32;
constexpr int CF_CNT_GLOBAL = CF_CNT_BASE + 20 * CF_CNT_STRIDE, CF_CNT_FLAG = CF_CNT_BASE + 21 * CF_CNT_STRIDE;
constexpr int CF_CNT_INTS = CF_CNT_BASE + 22 * CF_CNT_STRIDE;

// Grid-wide fixed-order reduction of the CTA partials into Gs (smem, fp64, upper) on every CTA,
// without grid barriers: the last CTA to arrive in each group of CF_FAN sums the group's
// partials (ws.gpart), the last group to finish sums the group sums into ws.G and bumps a
// generation flag; every CTA spins on the flag and reads the 528 packed entries.  The order of
// every sum is fixed (CTA order within a group, group order), so G is bitwise reproducible.
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ void cf_allreduce_gram(const CqArgs& a, double* Gs) {
    constexpr int NQ = (CF_NP + CF_THREADS - 1) / CF_THREADS;   // packed entries per thread
    constexpr int MAXG = (160 + CF_FAN - 1) / CF_FAN;           // grid <= 160 CTAs
    const int ngroups = (gridDim.x + CF_FAN - 1) / CF_FAN;
    const int grp = blockIdx.x / CF_FAN;
    const int gsize = min(CF_FAN, (int)gridDim.x - grp * CF_FAN);
    const int tid = threadIdx.x;
    int* cnt = a.ws.counters;
    unsigned* flag = reinterpret_cast<unsigned*>(cnt + CF_CNT_FLAG);
    __shared__ int s_last;
    __shared__ unsigned s_gen;
    if (tid == 0) s_gen = *(volatile unsigned*)flag;   // read before this CTA arrives
    fence_acq_rel_gpu();
    __syncthreads();
    int* gcnt = cnt + CF_CNT_BASE + grp * CF_CNT_STRIDE;
    if (tid == 0) s_last = (atomicAdd(gcnt, 1) == gsize - 1);
    __syncthreads();
#ifdef RG_CF_TRACE
    if (tid == 0) { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); cf_cta[3][blockIdx.x] = t; }
#endif
    if (s_last) {
        fence_acq_rel_gpu();
        const int c0 = grp * CF_FAN;
        double v[NQ][CF_FAN];
#pragma unroll
        for (int q = 0; q < NQ; ++q)
#pragma unroll
            for (int c = 0; c < CF_FAN; ++c) {
                const int e = tid + CF_THREADS * q;
                v[q][c] = (c < gsize && e < CF_NP) ? __ldcg(a.ws.part + (int64_t)(c0 + c) * CF_NP + e) : 0.0;
            }
#pragma unroll
        for (int q = 0; q < NQ; ++q) {
            const int e = tid + CF_THREADS * q;
            double sum = 0.0;
#pragma unroll
            for (int c = 0; c < CF_FAN; ++c) sum += v[q][c];
            if (e < CF_NP) a.ws.gpart[(int64_t)grp * CF_NP + e] = sum;
        }
        if (tid == 0) *gcnt = 0;
        fence_acq_rel_gpu();
        __syncthreads();
#ifdef RG_CF_TRACE
        if (tid == 0) { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); cf_cta[1][blockIdx.x] = t; }
#endif
        if (tid == 0) s_last = (atomicAdd(cnt + CF_CNT_GLOBAL, 1) == ngroups - 1);
        __syncthreads();
        if (s_last) {
            fence_acq_rel_gpu();
#pragma unroll
            for (int q = 0; q < NQ; ++q) {
                const int e = tid + CF_THREADS * q;
                if (e < CF_NP) {
                    double w[MAXG];
#pragma unroll
                    for (int g = 0; g < MAXG; ++g) w[g] = (g < ngroups) ? __ldcg(a.ws.gpart + (int64_t)g * CF_NP + e) : 0.0;
                    double sum = 0.0;
#pragma unroll
                    for (int g = 0; g < MAXG; ++g) sum += w[g];
                    a.ws.G[e] = sum;
                }
            }
            if (tid == 0) cnt[CF_CNT_GLOBAL] = 0;
            fence_acq_rel_gpu();
            __syncthreads();
#ifdef RG_CF_TRACE
            if (tid == 0) { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); cf_trace[8] = t; }
#endif
            if (tid == 0) atomicAdd(flag, 1u);
        }
    }
    if (tid == 0)
        while (ld_acquire_gpu(flag) == s_gen) __nanosleep(100);
    __syncthreads();
#ifdef RG_CF_TRACE
    if (tid == 0) { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); cf_cta[0][blockIdx.x] = t; }
#endif
    fence_acq_rel_gpu();
#pragma unroll
    for (int q = 0; q < NQ; ++q) {
        const int e = tid + CF_THREADS * q;
        if (e < CF_NP) {
            int i, j;
            tri_unpack(e, i, j);
            Gs[i + 32 * j] = __ldcg(a.ws.G + e);
        }
    }
    __syncthreads();
}

// tile (rows x 32, ld) <- tile * Rinv (32 x 32 fp32, [k * 32 + j]), chunks of 4 * CF_THREADS / 8 rows
__device__ void cf_times_rinv(float* tile, int ld, int rows, const float* Rinv) {
    constexpr int RG = CF_THREADS / 8;          // row groups x 8 column groups of 4
    const int tid = threadIdx.x;
    const int cgp = tid & 7, rgp = tid >> 3;
    for (int base = 0; base < rows; base += 4 * RG) {
        float o[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int c = 0; c < 4; ++c) o[i][c] = 0.f;
#pragma unroll 8
        for (int k = 0; k < CQ_NB; ++k) {
            const float4 rv = *reinterpret_cast<const float4*>(Rinv + k * 32 + 4 * cgp);
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


__global__ void __launch_bounds__(CF_THREADS, 1) cq_fused_kernel(CqArgs a, int ld) {
    RG_PDL_ENTRY();
    extern __shared__ __align__(16) uint8_t cf_smem[];
    float* tile = reinterpret_cast<float*>(cf_smem);
    double* sred = reinterpret_cast<double*>(cf_smem + (size_t)32 * ld * 4);
    double* Gs = sred + CF_SCR;               // 32 x CH_LD (first 1024 used as G)
    double* Rs = Gs + 32 * CH_LD;             // Cholesky scratch 32 x CH_LD
    float* Ri1 = reinterpret_cast<float*>(Rs + 32 * CH_LD);
    float* Ri2 = Ri1 + 1024;
    double* R1 = reinterpret_cast<double*>(Ri2 + 1024);
    __shared__ int s_flag[2];
    const int tid = threadIdx.x;
    CF_MARK(0);
    if (blockIdx.x == 0 && tid == 0) *a.ws.fail = 0;   // set again below only if a pivot fails
    const int64_t rows_per = (a.m + gridDim.x - 1) / gridDim.x;
    const int64_t r0 = (int64_t)blockIdx.x * rows_per;
    const int64_t rem = a.m - r0;
    const int rows = (int)(rem <= 0 ? 0 : (rem < rows_per ? rem : rows_per));
    // ---- load the CTA's rows (zero-padded columns beyond nc); 4 columns x CF_MAXPER rows of
    // independent loads in flight per thread
    for (int c0 = 0; c0 < 32; c0 += 4) {
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
    CF_MARK(1);
    // ---- pass 1: G1 = P^T P -> R1, R1^{-1} on every CTA
    cf_gram(tile, ld, rows, sred, a.ws.part + (int64_t)blockIdx.x * CF_NP);
    CF_MARK(2);
    CF_CTA(2);
    cf_allreduce_gram(a, Gs);
    CF_MARK(3);
    // sred is free after the Gram reduction: elimination scratch Y.  R^{-1} comes out row-major
    // ([k * 32 + j] = R^{-1}(k, j)), the layout cf_times_rinv reads.
    if (!chol_inv_cta<CF_THREADS, true>(Gs, a.nc, Rs, sred, R1, Ri1, true)) {
        if (blockIdx.x == 0 && tid == 0) *a.ws.fail = 1;   // the guarded MGS/TSQR kernels take over
        return;
    }
    CF_MARK(4);
    // kappa_F(R1) <= 2 nc  ->  single CholQR pass (see cq_pass_kernel)
    if (tid < 32) {
        double r = 0.0, ri = 0.0;
        for (int e = tid; e < 1024; e += 32) {
            const int i = e & 31, j = e >> 5;
            if (i < a.nc && j < a.nc) {
                r = fma(R1[e], R1[e], r);
                const double y = (double)Ri1[e];
                ri = fma(y, y, ri);
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            r += __shfl_xor_sync(0xffffffffu, r, o);
            ri += __shfl_xor_sync(0xffffffffu, ri, o);
        }
        if (tid == 0) s_flag[1] = (sqrt(r * ri) <= 2.0 * a.nc) ? 1 : 0;
    }
    __syncthreads();
    const bool single = s_flag[1] != 0;
    cf_times_rinv(tile, ld, rows, Ri1);   // tile <- Q1 = P R1^{-1}
    CF_MARK(5);
    if (!single) {
        // ---- pass 2: G2 = Q1^T Q1 -> R2 (left in Rs, row-major ld CH_LD), R2^{-1}; Q = Q1 R2^{-1}; R = R2 R1
        cf_gram(tile, ld, rows, sred, a.ws.part + (int64_t)blockIdx.x * CF_NP);
        cf_allreduce_gram(a, Gs);
        if (!chol_inv_cta<CF_THREADS, true>(Gs, a.nc, Rs, sred, nullptr, Ri2, true)) {
            if (blockIdx.x == 0 && tid == 0) *a.ws.fail = 1;
            return;   // input panel untouched in HBM: the MGS/TSQR fallback redoes it
        }
        cf_times_rinv(tile, ld, rows, Ri2);   // tile <- Q
        if (blockIdx.x == 0) {
            for (int e = tid; e < a.nc * a.nc; e += CF_THREADS) {
                const int i = e % a.nc, j = e / a.nc;
                double s = 0.0;
                for (int k = i; k <= j; ++k) s = fma(Rs[i * CH_LD + k], R1[k + 32 * j], s);
                a.Rout[i + (int64_t)j * a.ldr] = (i <= j) ? (float)s : 0.f;
            }
        }
    } else if (blockIdx.x == 0) {
        for (int e = tid; e < a.nc * a.nc; e += CF_THREADS) {
            const int i = e % a.nc, j = e / a.nc;
            a.Rout[i + (int64_t)j * a.ldr] = (i <= j) ? (float)R1[i + 32 * j] : 0.f;
        }
    }
    CF_MARK(6);
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
}

// distributed mode: after the host allreduce of G (pass `pass`), factor it (one warp)
__global__ void cq_factor_kernel(CqArgs a, int pass) {
    RG_PDL_ENTRY();
    __shared__ __align__(16) double Rs[32 * CH_LD];
    __shared__ __align__(16) double R1s[32 * CH_LD];
    if (pass > 0 && *(volatile int*)a.ws.fail) return;
    const bool ok = chol_inv_cta<256, false>(a.ws.G + pass * 1024, a.nc, Rs, R1s, a.ws.R + pass * 1024,
                                             a.ws.Rinv + pass * 1024, false);
    if (!ok && threadIdx.x == 0) *a.ws.fail = 1;
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
    const int grid = std::max(cq_grid(m), 160);   // also covers the fused kernel (<= 160 CTAs)
    const int ngroups = (grid + CQ_FAN - 1) / CQ_FAN + (grid + CF_FAN - 1) / CF_FAN;
    return (size_t)(grid + ngroups) * 1024 + 4 * 1024 + 1024 /*Rinv fp32 x2*/ + 64;
}

size_t cholqr_counter_ints(int64_t m) {
    const int grid = cq_grid(m);
    return std::max((size_t)(grid + CQ_FAN - 1) / CQ_FAN + 2, (size_t)CF_CNT_INTS);
}

cudaError_t launch_panel_cholqr(const CholqrLaunch& L, cudaStream_t st) {
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
    cudaError_t e;
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    }
    const int64_t rows_per = (L.m + sms - 1) / sms;
    if (!a.distributed && rows_per <= CF_MAX_ROWS && getenv("RGSQR_CQ_STREAM") == nullptr) {
        const int ld = (int)(rows_per | 1);   // odd leading dimension: conflict-free column walks
        const size_t smem = CfSmem::bytes(ld);
        static size_t attr = 0;
        if (smem > attr) {
            e = cudaFuncSetAttribute(cq_fused_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            if (e != cudaSuccess) return e;
            attr = smem;
        }
        // partial buffers: sms CTA partials + ceil(sms / 8) group partials fit in the workspace
        a.ws.gpart = a.ws.part + (size_t)sms * 1024;
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(sms);
        cfg.blockDim = dim3(CF_THREADS);
        cfg.dynamicSmemBytes = smem;
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeCooperative;
        at[0].val.cooperative = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        ++g_launches;
        return cudaLaunchKernelEx(&cfg, cq_fused_kernel, a, ld);
    }
    for (int pass = 0; pass < 3; ++pass) {
        if (pass == 0) RG_LAUNCH((cq_pass_kernel<0>), grid, CQ_THREADS, 0, st, a);
        if (pass == 1) RG_LAUNCH((cq_pass_kernel<1>), grid, CQ_THREADS, 0, st, a);
        if (pass == 2) RG_LAUNCH((cq_pass_kernel<2>), grid, CQ_THREADS, 0, st, a);
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

}  // namespace rg
