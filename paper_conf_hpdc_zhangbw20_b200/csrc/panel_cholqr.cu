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
// One warp.  G (32x32 fp64, upper triangle valid, nc x nc used, identity-padded).
// Writes R (fp64 upper, R[i + 32 j]) and Rinv (fp32, Rinv[i + 32 j]); returns false if a
// pivot is not safely positive (relative to the original diagonal).
template <bool kSharedG = false>
__device__ bool chol_inv_warp(const double* G, int nc, double* Rg, float* Rinvg, double* Rs /*smem 32x33*/) {
    __shared__ double dinv[32];
    const int lane = threadIdx.x & 31;
    double g[32];   // lane i holds row i of the symmetric Gram
#pragma unroll
    for (int j = 0; j < 32; ++j) {
        const int a = min(lane, j), b = max(lane, j);
        g[j] = (lane < nc && j < nc) ? (kSharedG ? G[a + 32 * b] : __ldcg(G + a + 32 * b)) : (lane == j ? 1.0 : 0.0);
    }
    double orig = 0.0;
#pragma unroll
    for (int j = 0; j < 32; ++j)
        if (j == lane) orig = g[j];
    bool ok = true;
    // Right-looking Cholesky; the pivot chain is kept short: lane k+1 forms its own next pivot
    // g(k+1,k+1) - R(k,k+1)^2 from its private row, and only that value crosses lanes.
    double dkk = __shfl_sync(0xffffffffu, g[0], 0);
#pragma unroll
    for (int k = 0; k < 32; ++k) {
        const double okk = __shfl_sync(0xffffffffu, orig, k);
        const bool good = (dkk > okk * 1e-15) && isfinite(dkk);
        ok = ok && good;
        const double irk = good ? rsqrt(dkk) : 1.0;
        const double rkk = good ? dkk * irk : 1.0;
        if (lane == k) dinv[k] = irk;
        // l = R(k, lane): row k of the upper factor
        const double l = (lane > k) ? g[k] * irk : ((lane == k) ? rkk : 0.0);
        if (k + 1 < 32) dkk = __shfl_sync(0xffffffffu, fma(-l, l, g[k + 1]), k + 1);
        Rs[k * 33 + lane] = l;
        __syncwarp();
#pragma unroll
        for (int j = k + 1; j < 32; ++j) g[j] = fma(-l, Rs[k * 33 + j], g[j]);
    }
    __syncwarp();
    // Rinv column j (= lane): x = e_j; for k = 31..0: x_k *= 1/R(k,k); x_i -= R(i,k) x_k (i < k)
    const int j = lane;
    double x[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) x[i] = (i == j) ? 1.0 : 0.0;
#pragma unroll
    for (int k = 31; k >= 0; --k) {
        x[k] *= dinv[k];
#pragma unroll
        for (int i = 0; i < k; ++i) x[i] = fma(-Rs[i * 33 + k], x[k], x[i]);
    }
    // coalesced stores: transpose through smem (Rs is no longer needed after this point)
#pragma unroll
    for (int i = 0; i < 32; ++i) Rg[i + 32 * j] = (i <= j) ? Rs[i * 33 + j] : 0.0;
    __syncwarp();
#pragma unroll
    for (int i = 0; i < 32; ++i) Rs[j * 33 + i] = x[i];   // Rs[j][i] = Rinv(i, j)
    __syncwarp();
#pragma unroll
    for (int jj = 0; jj < 32; ++jj) Rinvg[lane + 32 * jj] = (float)Rs[jj * 33 + lane];
    __syncwarp();
    return __all_sync(0xffffffffu, ok);
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
// R2 is in smem (Rs[i * 33 + j], from chol_inv_warp), R1 in the workspace.
__device__ void final_r_product(const CqArgs& a, const double* Rs, double* R1s /*smem 32x33*/) {
    for (int e = threadIdx.x; e < 1024; e += blockDim.x) R1s[(e & 31) * 33 + (e >> 5)] = __ldcg(a.ws.R + e);
    __syncthreads();
    for (int e = threadIdx.x; e < a.nc * a.nc; e += blockDim.x) {
        const int i = e % a.nc, j = e / a.nc;
        double s = 0.0;
        for (int k = i; k <= j; ++k) s = fma(Rs[i * 33 + k], R1s[k * 33 + j], s);
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
    __shared__ int s_ok;
    if (threadIdx.x < 32) {
        const bool ok = chol_inv_warp(G, a.nc, a.ws.R + pass * 1024, a.ws.Rinv + pass * 1024, smem_R);
        if (threadIdx.x == 0) {
            s_ok = ok;
            if (!ok) *a.ws.fail = 1;
        }
    }
    __syncthreads();
    if (pass == 0 && s_ok) single_pass_decision(a);
    if (pass == 1 && s_ok) final_r_product(a, smem_R, smem_R1);
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
    __shared__ double sred[2][1024];   // CTA partial-sum scratch (2 row groups at a time); reused
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
constexpr int CF_THREADS = 256;                  // 255 registers/thread: the Cholesky warp keeps 64 fp64 values
constexpr int CF_GROUPS = CF_THREADS / CQ_BLK;   // 7 row groups of 36 threads
constexpr int CF_FAN = 8;                        // CTA partials per first-level group
constexpr int CF_MAX_ROWS = 1408;                // rows per CTA that fit next to the scratch

struct CfSmem {
    static size_t bytes(int ld) {
        return (size_t)32 * ld * 4        // tile (column-major, ld)
               + 2 * 1024 * 8             // sred
               + 32 * 33 * 8 * 2          // G (padded) + Cholesky scratch
               + 2 * 32 * 32 * 4          // R1^{-1}, R2^{-1} (fp32, [k][j])
               + 1024 * 8                 // R1 (fp64) kept for R = R2 R1
               + 256;
    }
};

// Gram partial of the CTA's tile rows [0, rows) -> out (fp64 upper triangle), fixed order.
__device__ void cf_gram(const float* tile, int ld, int rows, double* sred, double* out_partial) {
    const int tid = threadIdx.x;
    const int g = tid / CQ_BLK, blk = tid % CQ_BLK;
    int bi = 0, bj = 0;
    blk_coords(blk, bi, bj);
    double acc[4][4] = {};
    if (g < CF_GROUPS) {
        for (int r = g; r < rows; r += CF_GROUPS) {
            double x[4], y[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                x[u] = (double)tile[(bi * 4 + u) * ld + r];
                y[u] = (double)tile[(bj * 4 + u) * ld + r];
            }
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int v = 0; v < 4; ++v) acc[u][v] = fma(x[u], y[v], acc[u][v]);
        }
    }
    for (int round = 0; round < (CF_GROUPS + 1) / 2; ++round) {
        const int g0 = round * 2;
        __syncthreads();
        for (int e = tid; e < 2 * 1024; e += CF_THREADS) sred[e] = 0.0;
        __syncthreads();
        if (g >= g0 && g < g0 + 2 && g < CF_GROUPS) {
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int v = 0; v < 4; ++v) sred[(g - g0) * 1024 + (bi * 4 + u) + (bj * 4 + v) * 32] = acc[u][v];
        }
        __syncthreads();
        for (int e = tid; e < 1024; e += CF_THREADS) {
            const int i = e & 31, j = e >> 5;
            double s = (round == 0) ? 0.0 : out_partial[e];
            s += sred[e] + sred[1024 + e];
            out_partial[e] = (i <= j) ? s : 0.0;
        }
    }
    __syncthreads();
}

// Grid-wide fixed-order reduction of the CTA partials into Gs (smem, fp64, upper) on every CTA.
__device__ void cf_allreduce_gram(const CqArgs& a, cg::grid_group& grid, double* Gs) {
    const int ngroups = (gridDim.x + CF_FAN - 1) / CF_FAN;
    grid.sync();
    if ((int)blockIdx.x < ngroups) {
        const int c0 = blockIdx.x * CF_FAN;
        const int cn = min(CF_FAN, (int)gridDim.x - c0);
        for (int e = threadIdx.x; e < 1024; e += CF_THREADS) {
            double v[CF_FAN];
#pragma unroll
            for (int c = 0; c < CF_FAN; ++c) v[c] = (c < cn) ? __ldcg(a.ws.part + (int64_t)(c0 + c) * 1024 + e) : 0.0;
            double sum = 0.0;
#pragma unroll
            for (int c = 0; c < CF_FAN; ++c) sum += v[c];
            a.ws.gpart[(int64_t)blockIdx.x * 1024 + e] = sum;
        }
    }
    grid.sync();
    for (int e = threadIdx.x; e < 1024; e += CF_THREADS) {
        double sum = 0.0;
        for (int g0 = 0; g0 < ngroups; g0 += CF_FAN) {
            double v[CF_FAN];
#pragma unroll
            for (int c = 0; c < CF_FAN; ++c) v[c] = (g0 + c < ngroups) ? __ldcg(a.ws.gpart + (int64_t)(g0 + c) * 1024 + e) : 0.0;
#pragma unroll
            for (int c = 0; c < CF_FAN; ++c) sum += v[c];
        }
        Gs[e] = sum;
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

__global__ void __launch_bounds__(CF_THREADS, 1) cq_fused_kernel(CqArgs a, int ld) {
    RG_PDL_ENTRY();
    cg::grid_group grid = cg::this_grid();
    extern __shared__ __align__(16) uint8_t cf_smem[];
    float* tile = reinterpret_cast<float*>(cf_smem);
    double* sred = reinterpret_cast<double*>(cf_smem + (size_t)32 * ld * 4);
    double* Gs = sred + 2 * 1024;             // 32 x 33 (first 1024 used as G)
    double* Rs = Gs + 32 * 33;                // Cholesky scratch 32 x 33
    float* Ri1 = reinterpret_cast<float*>(Rs + 32 * 33);
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
    // ---- load the CTA's rows (zero-padded columns beyond nc)
    for (int e = tid; e < 32 * rows; e += CF_THREADS) {
        const int r = e % rows, c = e / rows;
        tile[c * ld + r] = (c < a.nc) ? a.P[r0 + r + (int64_t)c * a.ldp] : 0.f;
    }
    __syncthreads();
    CF_MARK(1);
    // ---- pass 1: G1 = P^T P -> R1, R1^{-1} on every CTA
    cf_gram(tile, ld, rows, sred, a.ws.part + (int64_t)blockIdx.x * 1024);
    CF_MARK(2);
    cf_allreduce_gram(a, grid, Gs);
    CF_MARK(3);
    if (tid < 32) {
        const bool ok = chol_inv_warp<true>(Gs, a.nc, R1, Ri1, Rs);
        if (tid == 0) s_flag[0] = ok;
    }
    __syncthreads();
    CF_MARK(4);
    if (!s_flag[0]) {
        if (blockIdx.x == 0 && tid == 0) *a.ws.fail = 1;   // the guarded MGS/TSQR kernels take over
        return;
    }
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
    // Ri1 is [i + 32 j] (column-major R^{-1}); the product wants [k * 32 + j] = R^{-1}(k, j): transpose
    for (int e = tid; e < 1024; e += CF_THREADS) Ri2[e] = Ri1[(e >> 5) + 32 * (e & 31)];
    __syncthreads();
    cf_times_rinv(tile, ld, rows, Ri2);   // tile <- Q1 = P R1^{-1}
    CF_MARK(5);
    if (!single) {
        // ---- pass 2: G2 = Q1^T Q1 -> R2, R2^{-1}; Q = Q1 R2^{-1}; R = R2 R1
        cf_gram(tile, ld, rows, sred, a.ws.part + (int64_t)blockIdx.x * 1024);
        cf_allreduce_gram(a, grid, Gs);
        if (tid < 32) {   // R2 (fp64, [i + 32 j]) goes to sred, free after the reduction
            const bool ok = chol_inv_warp<true>(Gs, a.nc, sred, Ri1, Rs);
            if (tid == 0) s_flag[0] = ok;
        }
        __syncthreads();
        if (!s_flag[0]) {
            if (blockIdx.x == 0 && tid == 0) *a.ws.fail = 1;
            return;   // input panel untouched in HBM: the MGS/TSQR fallback redoes it
        }
        for (int e = tid; e < 1024; e += CF_THREADS) Ri2[e] = Ri1[(e >> 5) + 32 * (e & 31)];
        __syncthreads();
        cf_times_rinv(tile, ld, rows, Ri2);   // tile <- Q
        if (blockIdx.x == 0) {
            const double* R2 = reinterpret_cast<const double*>(sred);
            for (int e = tid; e < a.nc * a.nc; e += CF_THREADS) {
                const int i = e % a.nc, j = e / a.nc;
                double s = 0.0;
                for (int k = i; k <= j; ++k) s = fma(R2[i + 32 * k], R1[k + 32 * j], s);
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
    for (int e = tid; e < a.nc * rows; e += CF_THREADS) {
        const int r = e % rows, c = e / rows;
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

// distributed mode: after the host allreduce of G (pass `pass`), factor it (one warp)
__global__ void cq_factor_kernel(CqArgs a, int pass) {
    RG_PDL_ENTRY();
    __shared__ double Rs[32 * 33];
    __shared__ double R1s[32 * 33];
    __shared__ int s_ok;
    if (pass > 0 && *(volatile int*)a.ws.fail) return;
    if (threadIdx.x < 32) {
        const bool ok = chol_inv_warp(a.ws.G + pass * 1024, a.nc, a.ws.R + pass * 1024, a.ws.Rinv + pass * 1024, Rs);
        if (threadIdx.x == 0) {
            s_ok = ok;
            if (!ok) *a.ws.fail = 1;
        }
    }
    __syncthreads();
    if (pass == 0 && s_ok) single_pass_decision(a);
    if (pass == 1 && s_ok) final_r_product(a, Rs, R1s);
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
    return (size_t)(grid + CQ_FAN - 1) / CQ_FAN + 2;
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
