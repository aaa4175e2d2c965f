// sgemm.cu -- fp32 SIMT (no tensor core) forms of Algorithm 1's two trailing products, for the
// paper's Figure 7 ablation (section 4.1.2: "The third bar disables TensorCore") and
// the Table 3 SGEMM rows.  Development switch RGSQR_NO_TC=1; not the product path.
//   K1:  R12 = Q1^T A2   (h x w, contraction over the m rows; split-K partials + fixed-order sum)
//   K2:  A2 <- A2 - Q1 R12
// Register-blocked 64 x 64 output tiles, 256 threads (4 x 4 outputs each), 16-row (K1) / 16-column
// (K2) slabs staged in shared memory.
#include <cuda_runtime.h>

#include <algorithm>

#include "kernels.h"

namespace rg {

constexpr int SG_T = 64;   // output tile
constexpr int SG_K = 16;   // contraction slab

// P[split][j * h + i] = sum_{r in split} Q1(r, i) A2(r, j)
__global__ void __launch_bounds__(256) sgemm_tn_kernel(const float* __restrict__ Q1, const float* __restrict__ A2,
                                                       int64_t ld, int64_t m, int h, int w, int64_t rows_per,
                                                       float* __restrict__ P) {
    __shared__ float sa[SG_K][SG_T + 4], sb[SG_K][SG_T + 4];
    const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
    const int i0 = blockIdx.x * SG_T, j0 = blockIdx.y * SG_T;
    const int64_t r0 = (int64_t)blockIdx.z * rows_per, r1 = min(m, r0 + rows_per);
    float acc[4][4] = {};
    for (int64_t k0 = r0; k0 < r1; k0 += SG_K) {
        for (int e = threadIdx.x; e < SG_K * SG_T; e += 256) {
            const int kk = e % SG_K, c = e / SG_K;   // consecutive threads walk the rows of a column
            const int64_t r = k0 + kk;
            sa[kk][c] = (r < r1 && i0 + c < h) ? Q1[r + (int64_t)(i0 + c) * ld] : 0.f;
            sb[kk][c] = (r < r1 && j0 + c < w) ? A2[r + (int64_t)(j0 + c) * ld] : 0.f;
        }
        __syncthreads();
#pragma unroll
        for (int kk = 0; kk < SG_K; ++kk) {
            float a[4], b[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                a[u] = sa[kk][ty + 16 * u];
                b[u] = sb[kk][tx + 16 * u];
            }
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int v = 0; v < 4; ++v) acc[u][v] = fmaf(a[u], b[v], acc[u][v]);
        }
        __syncthreads();
    }
    float* out = P + (int64_t)blockIdx.z * h * w;
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            const int i = i0 + ty + 16 * u, j = j0 + tx + 16 * v;
            if (i < h && j < w) out[(int64_t)j * h + i] = acc[u][v];
        }
}

// R(i, j) = sum_s P[s][j * h + i] (fixed order)
__global__ void sgemm_reduce_kernel(const float* __restrict__ P, int splits, int h, int w, float* __restrict__ R,
                                    int64_t ldr) {
    const int64_t total = (int64_t)h * w;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        float s = 0.f;
        for (int z = 0; z < splits; ++z) s += P[(int64_t)z * total + e];
        R[(e % h) + (e / h) * ldr] = s;
    }
}

// A2(r, j) -= sum_i Q1(r, i) R12(i, j)
__global__ void __launch_bounds__(256) sgemm_nn_update_kernel(const float* __restrict__ Q1, const float* __restrict__ R12,
                                                              int64_t ldr, float* __restrict__ A2, int64_t ld, int64_t m,
                                                              int h, int w) {
    __shared__ float sa[SG_K][SG_T + 4], sb[SG_K][SG_T + 4];
    const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
    const int64_t r0 = (int64_t)blockIdx.x * SG_T;
    const int j0 = blockIdx.y * SG_T;
    float acc[4][4] = {};
    for (int k0 = 0; k0 < h; k0 += SG_K) {
        for (int e = threadIdx.x; e < SG_K * SG_T; e += 256) {
            const int rr = e % SG_T, kk = e / SG_T;
            sa[kk][rr] = (r0 + rr < m && k0 + kk < h) ? Q1[r0 + rr + (int64_t)(k0 + kk) * ld] : 0.f;
            const int c = e % SG_T;
            sb[kk][c] = (k0 + kk < h && j0 + c < w) ? R12[(k0 + kk) + (int64_t)(j0 + c) * ldr] : 0.f;
        }
        __syncthreads();
#pragma unroll
        for (int kk = 0; kk < SG_K; ++kk) {
            float a[4], b[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                a[u] = sa[kk][tx + 16 * u];
                b[u] = sb[kk][ty + 16 * u];
            }
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int v = 0; v < 4; ++v) acc[u][v] = fmaf(a[u], b[v], acc[u][v]);
        }
        __syncthreads();
    }
#pragma unroll
    for (int v = 0; v < 4; ++v) {
        const int j = j0 + ty + 16 * v;
        if (j >= w) continue;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int64_t r = r0 + tx + 16 * u;
            if (r < m) A2[r + (int64_t)j * ld] -= acc[u][v];
        }
    }
}

size_t sgemm_tn_work_floats(int64_t m, int h, int w) {
    const int64_t tiles = (int64_t)((h + SG_T - 1) / SG_T) * ((w + SG_T - 1) / SG_T);
    const int64_t splits = std::max<int64_t>(1, std::min<int64_t>((148 * 4 + tiles - 1) / tiles, (m + 255) / 256));
    return (size_t)splits * h * w;
}

cudaError_t launch_sgemm_proj(const float* Q1, const float* A2, int64_t ld, int64_t m, int h, int w, float* R,
                              int64_t ldr, float* work, cudaStream_t st) {
    const int ti = (h + SG_T - 1) / SG_T, tj = (w + SG_T - 1) / SG_T;
    const int64_t tiles = (int64_t)ti * tj;
    int64_t splits = std::max<int64_t>(1, std::min<int64_t>((148 * 4 + tiles - 1) / tiles, (m + 255) / 256));
    const int64_t rows_per = ((m + splits - 1) / splits + SG_K - 1) / SG_K * SG_K;
    splits = (m + rows_per - 1) / rows_per;
    RG_LAUNCH((sgemm_tn_kernel), dim3(ti, tj, (unsigned)splits), 256, 0, st, Q1, A2, ld, m, h, w, rows_per, work);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    const int64_t total = (int64_t)h * w;
    RG_LAUNCH((sgemm_reduce_kernel), (unsigned)std::min<int64_t>((total + 255) / 256, 148 * 8), 256, 0, st, work,
              (int)splits, h, w, R, ldr);
    return cudaGetLastError();
}

cudaError_t launch_sgemm_update(const float* Q1, const float* R12, int64_t ldr, float* A2, int64_t ld, int64_t m, int h,
                                int w, cudaStream_t st) {
    dim3 grid((unsigned)((m + SG_T - 1) / SG_T), (unsigned)((w + SG_T - 1) / SG_T));
    RG_LAUNCH((sgemm_nn_update_kernel), grid, 256, 0, st, Q1, R12, ldr, A2, ld, m, h, w);
    return cudaGetLastError();
}

}  // namespace rg
