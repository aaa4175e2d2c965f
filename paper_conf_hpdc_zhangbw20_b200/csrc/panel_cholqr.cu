// panel_cholqr.cu -- CholQR2 leaf panel with an fp64 Gram matrix (north_star: "a
// bandwidth-bound panel MGS/CholQR kernel"; SURVEY 2.2 A19/8(e) "CholQR2 (fp64 Gram)").
//
//   G1 = P^T P (fp64)          R1 = chol(G1)     Q1 = P R1^{-1}   (fp32)
//   G2 = Q1^T Q1 (fp64)        R2 = chol(G2)     Q  = Q1 R2^{-1}  (fp32 + 16-bit shadow)
//   R  = R2 R1
//
// Why it replaces the MGS tiles by default on B200: MGS needs 32
// dependent block-wide reductions per tile plus a tree of stacked-R factorizations, which
// is latency-bound (~240 us per 65536 x 32 panel measured); CholQR2 is three streaming
// passes whose only sequential piece is a 32 x 32 Cholesky done redundantly per CTA.
// With an fp64 Gram, Q1's orthogonality is ~kappa u32 (like MGS) and the second pass
// brings it to ~u32 while kappa(P) < ~1e7.  If a Cholesky pivot fails the panel sets a
// device flag and the MGS/TSQR kernels of panel.cu (guarded by that flag) redo the panel
// from the untouched input, so the result never silently degrades.
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>

#include "kernels.h"

namespace rg {

constexpr int CQ_NB = 32;
constexpr int CQ_TILE = 128;          // rows staged per iteration
constexpr int CQ_LD = CQ_TILE + 1;    // smem column stride (bank-conflict-free column access)
constexpr int CQ_THREADS = 256;
constexpr int CQ_BLK = 36;            // 4x4 blocks in the upper triangle of a 32x32 Gram (8*9/2)
constexpr int CQ_GROUPS = CQ_THREADS / CQ_BLK;  // 7 row groups of 36 threads

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

struct CqArgs {
    const float* P;     // panel input (fp32, ldp)
    int64_t ldp;
    float* Q1;          // pass-1 output (workspace, ld = m)
    float* Q;           // final Q (in place of the panel is allowed), ldq
    int64_t ldq;
    uint16_t* Qh;       // 16-bit shadow (hi) of Q, ldh
    uint16_t* Ql;       // lo part (split mode) or null
    int64_t ldh;
    int64_t m;
    int nc;
    double* part;       // per-CTA partial Grams [grid][32*32]
    double* G;          // reduced Gram (32*32, fp64), pass 1 at G, pass 2 at G + 1024
    double* Rkeep;      // R1 (fp64 32*32) kept for the final product
    int* counter;       // last-block counter (reset by the last block)
    int* fail;          // set to 1 when a Cholesky pivot fails (MGS fallback runs)
    float* R;           // final nc x nc R block (ldr)
    int64_t ldr;
    int bf16;
    int distributed;    // 1: the caller allreduces G between passes (no last-block reduce)
};

// Accumulate the 4x4 Gram block `blk` of the nc-column tile in smem (rows [0, rows)).
__device__ __forceinline__ void gram_block_accum(const float* tile, int rows, int g, int blk, double (&acc)[4][4]) {
    // upper-triangular block (bi, bj), bi <= bj, enumerated row-major
    int bi = 0, rem = blk;
    while (rem >= 8 - bi) {
        rem -= 8 - bi;
        ++bi;
    }
    const int bj = bi + rem;
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

__device__ __forceinline__ void gram_block_store(double* dst, int blk, const double (&acc)[4][4]) {
    int bi = 0, rem = blk;
    while (rem >= 8 - bi) {
        rem -= 8 - bi;
        ++bi;
    }
    const int bj = bi + rem;
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) dst[(bi * 4 + u) + (bj * 4 + v) * 32] = acc[u][v];
}

// Sum the per-group partial blocks of this CTA (smem) and write the CTA partial Gram.
__device__ void cta_gram_flush(double* sred, const double (&acc)[4][4], int blk, int g, double* out) {
    // sred: [CQ_GROUPS][1024] doubles
    if (blk < CQ_BLK && g < CQ_GROUPS) gram_block_store(sred + g * 1024, blk, acc);
    __syncthreads();
    for (int e = threadIdx.x; e < 1024; e += blockDim.x) {
        double s = 0.0;
        for (int q = 0; q < CQ_GROUPS; ++q) s += sred[q * 1024 + e];
        out[e] = s;   // only the upper triangle is meaningful
    }
}

// last CTA sums all CTA partials in fixed order into G (fp64, symmetric fill)
__device__ bool last_block_reduce(const CqArgs& a, double* Gout) {
    __shared__ int s_last;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) {
        const int old = atomicAdd(a.counter, 1);
        s_last = (old == (int)gridDim.x - 1);
    }
    __syncthreads();
    if (!s_last) return false;
    __threadfence();
    for (int e = threadIdx.x; e < 1024; e += blockDim.x) {
        const int i = e & 31, j = e >> 5;
        double s = 0.0;
        if (i <= j)
            for (int c = 0; c < (int)gridDim.x; ++c) s += __ldcg(a.part + (int64_t)c * 1024 + e);
        Gout[e] = s;
    }
    __syncthreads();
    if (threadIdx.x == 0) *a.counter = 0;
    return true;
}

// Cholesky G = R^T R (upper R, fp64) of the nc x nc leading block, padded with identity,
// by warp 0; then Rinv = R^{-1} (fp64).  Returns false (all threads) on a failed pivot.
__device__ bool chol_inv(const double* Gg, double* Rs /*32x33*/, double* Ri /*32x33*/, int nc) {
    __shared__ int s_ok;
    const int lane = threadIdx.x & 31;
    if (threadIdx.x < 32) {
        // load the upper triangle (column j in lane j's view): Rs[i][j] = G(i, j) for i <= j
        for (int i = 0; i < 32; ++i) {
            const int j = lane;
            double v = 0.0;
            if (i < nc && j < nc) v = (i <= j) ? Gg[i + j * 32] : 0.0;
            else if (i == j) v = 1.0;
            Rs[i * 33 + j] = (i <= j) ? v : 0.0;
        }
        __syncwarp();
        bool ok = true;
        // right-looking upper Cholesky: for k: R(k,k) = sqrt(G(k,k)); R(k,j) /= R(k,k);
        // G(i,j) -= R(k,i) R(k,j) for k < i <= j.  Lane j owns column j.
        for (int k = 0; k < 32; ++k) {
            const double piv = Rs[k * 33 + k];
            const double orig = (k < nc) ? Gg[k + k * 32] : 1.0;
            const bool good = piv > orig * 1e-15 && isfinite(piv);
            ok = ok && good;
            const double d = good ? sqrt(piv) : 1.0;
            __syncwarp();
            if (lane >= k) Rs[k * 33 + lane] = (lane == k) ? d : Rs[k * 33 + lane] / d;
            __syncwarp();
            const double rkj = Rs[k * 33 + lane];
            for (int i = k + 1; i <= lane; ++i) Rs[i * 33 + lane] -= Rs[k * 33 + i] * rkj;
            __syncwarp();
        }
        // Rinv by column-oriented back substitution: lane j solves R x = e_j
        for (int i = 0; i < 32; ++i) Ri[i * 33 + lane] = 0.0;
        __syncwarp();
        {
            const int j = lane;
            double x[32];
#pragma unroll
            for (int i = 0; i < 32; ++i) x[i] = (i == j) ? 1.0 : 0.0;
#pragma unroll
            for (int k = 31; k >= 0; --k) {
                if (k <= j) {
                    x[k] = x[k] / Rs[k * 33 + k];
#pragma unroll
                    for (int i = 0; i < k; ++i) x[i] -= Rs[i * 33 + k] * x[k];
                }
            }
#pragma unroll
            for (int i = 0; i < 32; ++i) Ri[i * 33 + j] = (i <= j) ? x[i] : 0.0;
        }
        if (lane == 0) s_ok = ok ? 1 : 0;
    }
    __syncthreads();
    return s_ok != 0;
}

// pass 1: CTA partial Grams of P; last block reduces into G (unless distributed).
__global__ void __launch_bounds__(CQ_THREADS) cq_gram_kernel(CqArgs a) {
    extern __shared__ double dsm[];
    float* tile = reinterpret_cast<float*>(dsm + CQ_GROUPS * 1024);
    double* sred = dsm;
    const int tid = threadIdx.x;
    if (blockIdx.x == 0 && tid == 0) *a.fail = 0;   // the apply passes / MGS fallback read it later
    const int g = tid / CQ_BLK, blk = tid % CQ_BLK;
    double acc[4][4] = {};
    const int64_t rows_per_cta = (a.m + gridDim.x - 1) / gridDim.x;
    const int64_t r0 = (int64_t)blockIdx.x * rows_per_cta;
    const int64_t r1 = min(a.m, r0 + rows_per_cta);
    for (int64_t base = r0; base < r1; base += CQ_TILE) {
        const int rows = (int)((r1 - base) < CQ_TILE ? (r1 - base) : CQ_TILE);
        __syncthreads();
        for (int e = tid; e < CQ_TILE * CQ_NB; e += CQ_THREADS) {
            const int r = e % CQ_TILE, c = e / CQ_TILE;
            tile[c * CQ_LD + r] = (r < rows && c < a.nc) ? a.P[base + r + (int64_t)c * a.ldp] : 0.f;
        }
        __syncthreads();
        if (g < CQ_GROUPS) gram_block_accum(tile, rows, g, blk, acc);
    }
    __syncthreads();
    cta_gram_flush(sred, acc, blk, g, a.part + (int64_t)blockIdx.x * 1024);
    if (!a.distributed) last_block_reduce(a, a.G);
}

// pass 2 (mode 0): Q1 = P R1^{-1} + partial Grams of Q1 (last block -> G + 1024)
// pass 3 (mode 1): Q  = Q1 R2^{-1} (+ shadow), R = R2 R1
template <int MODE>
__global__ void __launch_bounds__(CQ_THREADS) cq_apply_kernel(CqArgs a) {
    extern __shared__ double dsm[];
    double* Rs = dsm;                    // 32 x 33
    double* Ri = Rs + 32 * 33;           // 32 x 33
    float* Rif = reinterpret_cast<float*>(Ri + 32 * 33);            // 32 x 33 fp32 R^{-1}
    double* sred = reinterpret_cast<double*>(Rif + 32 * 34);        // [CQ_GROUPS][1024]
    float* tile = reinterpret_cast<float*>(sred + CQ_GROUPS * 1024); // 32 x CQ_LD
    const int tid = threadIdx.x;
    if (*a.fail) return;   // an earlier pivot failed: the MGS fallback owns this panel
    const double* Gin = a.G + (MODE == 0 ? 0 : 1024);
    const bool ok = chol_inv(Gin, Rs, Ri, a.nc);
    if (!ok) {
        if (tid == 0) atomicExch(a.fail, 1);
        return;
    }
    for (int e = tid; e < 32 * 32; e += CQ_THREADS) {
        const int i = e & 31, j = e >> 5;
        Rif[i * 33 + j] = (float)Ri[i * 33 + j];
    }
    if (MODE == 0 && blockIdx.x == 0)
        for (int e = tid; e < 32 * 32; e += CQ_THREADS) a.Rkeep[e] = Rs[(e & 31) * 33 + (e >> 5)];
    if (MODE == 1 && blockIdx.x == 0) {
        // R = R2 R1 (fp64 product of upper-triangular factors, positive diagonal)
        for (int e = tid; e < a.nc * a.nc; e += CQ_THREADS) {
            const int i = e % a.nc, j = e / a.nc;
            double s = 0.0;
            for (int k = i; k <= j; ++k) s = fma(Rs[i * 33 + k], a.Rkeep[k + j * 32], s);
            a.R[i + (int64_t)j * a.ldr] = (i <= j) ? (float)s : 0.f;
        }
    }
    __syncthreads();
    const int g = tid / CQ_BLK, blk = tid % CQ_BLK;
    double acc[4][4] = {};
    const float* src = MODE == 0 ? a.P : a.Q1;
    const int64_t lds = MODE == 0 ? a.ldp : a.m;
    const int64_t rows_per_cta = (a.m + gridDim.x - 1) / gridDim.x;
    const int64_t r0 = (int64_t)blockIdx.x * rows_per_cta;
    const int64_t r1 = min(a.m, r0 + rows_per_cta);
    const int row = tid & (CQ_TILE - 1), half = tid >> 7;   // 2 threads per row: columns [16 half, 16 half + 16)
    for (int64_t base = r0; base < r1; base += CQ_TILE) {
        const int rows = (int)((r1 - base) < CQ_TILE ? (r1 - base) : CQ_TILE);
        __syncthreads();
        for (int e = tid; e < CQ_TILE * CQ_NB; e += CQ_THREADS) {
            const int r = e % CQ_TILE, c = e / CQ_TILE;
            tile[c * CQ_LD + r] = (r < rows && c < a.nc) ? src[base + r + (int64_t)c * lds] : 0.f;
        }
        __syncthreads();
        float out[16];
#pragma unroll
        for (int jj = 0; jj < 16; ++jj) out[jj] = 0.f;
        if (row < rows) {
#pragma unroll 4
            for (int k = 0; k < CQ_NB; ++k) {
                const float x = tile[k * CQ_LD + row];
#pragma unroll
                for (int jj = 0; jj < 16; ++jj) out[jj] = fmaf(x, Rif[k * 33 + half * 16 + jj], out[jj]);
            }
        }
        __syncthreads();
        if (row < rows) {
#pragma unroll
            for (int jj = 0; jj < 16; ++jj) {
                const int c = half * 16 + jj;
                if (c < a.nc) {
                    const int64_t gr = base + row;
                    if (MODE == 0) {
                        a.Q1[gr + (int64_t)c * a.m] = out[jj];
                        tile[c * CQ_LD + row] = out[jj];
                    } else {
                        a.Q[gr + (int64_t)c * a.ldq] = out[jj];
                        if (a.Qh) {
                            const uint16_t hb = cq_to16(out[jj], a.bf16);
                            a.Qh[gr + (int64_t)c * a.ldh] = hb;
                            if (a.Ql) a.Ql[gr + (int64_t)c * a.ldh] = cq_to16((out[jj] - cq_from16(hb, a.bf16)) * 2048.f,
                                                                             a.bf16);
                        }
                    }
                }
            }
        }
        if (MODE == 0) {
            __syncthreads();
            if (g < CQ_GROUPS) gram_block_accum(tile, rows, g, blk, acc);
        }
    }
    if (MODE == 0) {
        __syncthreads();
        cta_gram_flush(sred, acc, blk, g, a.part + (int64_t)blockIdx.x * 1024);
        if (!a.distributed) last_block_reduce(a, a.G + 1024);
    }
}

// distributed mode: sum the CTA partials (fixed order) into G (before the NCCL allreduce)
__global__ void cq_sum_parts_kernel(const double* __restrict__ part, int nparts, double* __restrict__ G) {
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= 1024) return;
    double s = 0.0;
    if ((e & 31) <= (e >> 5))
        for (int c = 0; c < nparts; ++c) s += part[(int64_t)c * 1024 + e];
    G[e] = s;
}

// ------------------------------------------------------------------ host side
static int cq_grid(int64_t m) {
    int64_t g = (m + 511) / 512;   // >= 512 rows per CTA keeps the per-CTA Cholesky amortised
    if (g > 148) g = 148;
    if (g < 1) g = 1;
    return (int)g;
}

size_t cholqr_ws_doubles(int64_t m) { return (size_t)cq_grid(m) * 1024 + 3 * 1024 + 64; }

cudaError_t launch_panel_cholqr(const CholqrLaunch& L, cudaStream_t st) {
    CqArgs a{};
    a.P = L.P;
    a.ldp = L.ldp;
    a.Q1 = L.Q1;
    a.Q = L.Q;
    a.ldq = L.ldq;
    a.Qh = L.Qh;
    a.Ql = L.Ql;
    a.ldh = L.ldh;
    a.m = L.m;
    a.nc = L.nc;
    const int grid = cq_grid(L.m);
    a.part = L.ws;
    a.G = L.ws + (size_t)grid * 1024;
    a.Rkeep = a.G + 2048;
    a.counter = L.counter;
    a.fail = L.fail;
    a.R = L.R;
    a.ldr = L.ldr;
    a.bf16 = L.bf16;
    a.distributed = L.allreduce_g != nullptr;
    const size_t smem1 = (size_t)CQ_GROUPS * 1024 * 8 + (size_t)32 * CQ_LD * 4;
    const size_t smem2 = (size_t)2 * 32 * 33 * 8 + 32 * 34 * 4 + (size_t)CQ_GROUPS * 1024 * 8 + (size_t)32 * CQ_LD * 4;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(cq_gram_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem1);
        cudaFuncSetAttribute(cq_apply_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem2);
        cudaFuncSetAttribute(cq_apply_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem2);
        attr = true;
    }
    ++g_launches;
    cq_gram_kernel<<<grid, CQ_THREADS, smem1, st>>>(a);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    if (a.distributed) {
        ++g_launches;
        cq_sum_parts_kernel<<<4, 256, 0, st>>>(a.part, grid, a.G);
        if (L.allreduce_g(a.G, L.ctx) != 0) return cudaErrorUnknown;
    }
    ++g_launches;
    cq_apply_kernel<0><<<grid, CQ_THREADS, smem2, st>>>(a);
    e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    if (a.distributed) {
        ++g_launches;
        cq_sum_parts_kernel<<<4, 256, 0, st>>>(a.part, grid, a.G + 1024);
        if (L.allreduce_g(a.G + 1024, L.ctx) != 0) return cudaErrorUnknown;
    }
    ++g_launches;
    cq_apply_kernel<1><<<grid, CQ_THREADS, smem2, st>>>(a);
    return cudaGetLastError();
}

}  // namespace rg
