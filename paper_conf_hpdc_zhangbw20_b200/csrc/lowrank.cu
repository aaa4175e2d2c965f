// lowrank.cu -- kernels of lowrank_approx (section 3.4; BASELINE
// config 5; reading #17): operand casts with power-of-two row scaling, and the one-sided
// Jacobi SVD of the small (rank + oversample)^2 triangular factor R_b.
//
// Jacobi (Hestenes): W = R_b, V = I; sweeps of the round-robin ("tournament") ordering,
// one warp per column pair (p, q): alpha = |w_p|^2, beta = |w_q|^2, gamma = w_p^T w_q,
// zeta = (beta - alpha) / (2 gamma), t = sign(zeta) / (|zeta| + sqrt(1 + zeta^2)),
// c = 1/sqrt(1 + t^2), s = c t, [w_p w_q] <- [w_p w_q] [c s; -s c] (same for V).
// fp64 throughout; a cooperative grid synchronises the rounds; converged when every
// |gamma| <= tol sqrt(alpha beta) during a sweep.  Singular values are the column norms.
#include <cooperative_groups.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>

#include "kernels.h"

namespace cg = cooperative_groups;

namespace rg {

__device__ __forceinline__ uint16_t lr_to16(float x, int bf16) {
    if (bf16) {
        __nv_bfloat16 b = __float2bfloat16_rn(x);
        return *reinterpret_cast<uint16_t*>(&b);
    }
    __half h = __float2half_rn(x);
    return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float lr_from16(uint16_t u, int bf16) {
    if (bf16) return __bfloat162float(*reinterpret_cast<__nv_bfloat16*>(&u));
    return __half2float(*reinterpret_cast<__half*>(&u));
}

// dst_hi/lo (rows x cols, ldd) = 16-bit images of src * (1 / rscale[i]) (fp32 or fp64 src).
// lo = 16-bit((x - hi) 2^11) when dst_lo is non-null (split precision, reading #9).
template <typename T>
__global__ void cast_rows_kernel(const T* __restrict__ src, int64_t lds, int64_t rows, int cols,
                                 const float* __restrict__ rscale, uint16_t* __restrict__ hi, uint16_t* __restrict__ lo,
                                 int64_t ldd, int bf16) {
    RG_PDL_ENTRY();
    const int64_t total = rows * cols;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = e % rows;
        const int64_t j = e / rows;
        float x = (float)src[i + j * lds];
        if (rscale) x = x / rscale[i];
        const uint16_t h = lr_to16(x, bf16);
        hi[i + j * ldd] = h;
        if (lo) lo[i + j * ldd] = lr_to16((x - lr_from16(h, bf16)) * 2048.f, bf16);
    }
}

// X(i, :) /= rscale[i] in place (undo a power-of-two row scaling)
__global__ void unscale_rows_kernel(float* __restrict__ X, int64_t ldx, int64_t rows, int cols,
                                    const float* __restrict__ rscale) {
    RG_PDL_ENTRY();
    const int64_t total = rows * cols;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = e % rows;
        const int64_t j = e / rows;
        X[i + j * ldx] /= rscale[i];   // powers of two: exact
    }
}

// W (l x l fp64, ld l) = R (upper fp32, ldr), V = I
__global__ void jacobi_init_kernel(const float* __restrict__ R, int64_t ldr, int l, double* __restrict__ W,
                                   double* __restrict__ V) {
    RG_PDL_ENTRY();
    const int64_t total = (int64_t)l * l;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int i = (int)(e % l), j = (int)(e / l);
        W[e] = (i <= j) ? (double)R[i + (int64_t)j * ldr] : 0.0;
        V[e] = (i == j) ? 1.0 : 0.0;
    }
}

__device__ __forceinline__ double wsum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// round-robin pairing of L (even) players, round r in [0, L-1), pair k in [0, L/2)
__device__ __forceinline__ void rr_pair(int L, int r, int k, int& p, int& q) {
    if (k == 0) {
        p = L - 1;
        q = r;
    } else {
        p = (r + k) % (L - 1);
        q = (r - k + (L - 1)) % (L - 1);
    }
    if (p > q) {
        const int t = p;
        p = q;
        q = t;
    }
}

// flags[0]: rotations above tolerance in the current sweep (int); flags[1]: sweeps done
__global__ void __launch_bounds__(256) jacobi_sweeps_kernel(double* __restrict__ W, double* __restrict__ V, int l,
                                                            int max_sweeps, double tol, int* flags) {
    RG_PDL_ENTRY();
    cg::grid_group grid = cg::this_grid();
    const int lane = threadIdx.x & 31;
    const int gwarp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int nwarps = (gridDim.x * blockDim.x) >> 5;
    const int L = (l + 1) & ~1;   // pad to even with a virtual zero column (index l)
    int sweep = 0;
    for (; sweep < max_sweeps; ++sweep) {
        if (gwarp == 0 && lane == 0) flags[0] = 0;
        grid.sync();
        for (int r = 0; r < L - 1; ++r) {
            for (int k = gwarp; k < L / 2; k += nwarps) {
                int p, q;
                rr_pair(L, r, k, p, q);
                if (q >= l) continue;   // pair with the virtual column: nothing to do
                double* wp = W + (int64_t)p * l;
                double* wq = W + (int64_t)q * l;
                double a = 0.0, b = 0.0, g = 0.0;
                for (int i = lane; i < l; i += 32) {
                    const double x = __ldcg(wp + i), y = __ldcg(wq + i);
                    a = fma(x, x, a);
                    b = fma(y, y, b);
                    g = fma(x, y, g);
                }
                a = wsum(a);
                b = wsum(b);
                g = wsum(g);
                if (fabs(g) <= tol * sqrt(a * b) || g == 0.0) continue;
                if (lane == 0) atomicAdd(&flags[0], 1);
                const double zeta = (b - a) / (2.0 * g);
                const double t = (zeta >= 0.0 ? 1.0 : -1.0) / (fabs(zeta) + sqrt(1.0 + zeta * zeta));
                const double c = 1.0 / sqrt(1.0 + t * t), s = c * t;
                double* vp = V + (int64_t)p * l;
                double* vq = V + (int64_t)q * l;
                for (int i = lane; i < l; i += 32) {
                    const double x = __ldcg(wp + i), y = __ldcg(wq + i);
                    wp[i] = c * x - s * y;
                    wq[i] = s * x + c * y;
                    const double u = __ldcg(vp + i), v = __ldcg(vq + i);
                    vp[i] = c * u - s * v;
                    vq[i] = s * u + c * v;
                }
            }
            grid.sync();
        }
        const int rotated = *(volatile int*)&flags[0];
        grid.sync();
        if (rotated == 0) {
            ++sweep;
            break;
        }
    }
    if (gwarp == 0 && lane == 0) flags[1] = sweep;
}

// sigma_j = |w_j|; rank by descending sigma (ties by index); for rank < r write
// S[rank], Ub[:, rank] = w_j / sigma_j (fp32, ld l), Vb[:, rank] = v_j (fp32, ld l).
__global__ void jacobi_extract_kernel(const double* __restrict__ W, const double* __restrict__ V, int l, int r,
                                      float* __restrict__ S, float* __restrict__ Ub, float* __restrict__ Vb,
                                      double* __restrict__ sig) {
    RG_PDL_ENTRY();
    // one CTA per column j
    const int j = blockIdx.x;
    __shared__ double red[32];
    __shared__ int s_rank;
    const double* w = W + (int64_t)j * l;
    double a = 0.0;
    for (int i = threadIdx.x; i < l; i += blockDim.x) a = fma(w[i], w[i], a);
    a = wsum(a);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = a;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int k = 0; k < (int)(blockDim.x >> 5); ++k) t += red[k];
        sig[j] = sqrt(t);
    }
}

__global__ void jacobi_rank_kernel(const double* __restrict__ W, const double* __restrict__ V, int l, int r,
                                   const double* __restrict__ sig, float* __restrict__ S, float* __restrict__ Ub,
                                   float* __restrict__ Vb) {
    RG_PDL_ENTRY();
    const int j = blockIdx.x;
    __shared__ int s_rank;
    if (threadIdx.x == 0) {
        const double sj = sig[j];
        int rank = 0;
        for (int i = 0; i < l; ++i) {
            const double si = sig[i];
            rank += (si > sj) || (si == sj && i < j);
        }
        s_rank = rank;
    }
    __syncthreads();
    const int rank = s_rank;
    if (rank >= r) return;
    const double sj = sig[j];
    if (threadIdx.x == 0) S[rank] = (float)sj;
    const double inv = sj > 0.0 ? 1.0 / sj : 0.0;
    for (int i = threadIdx.x; i < l; i += blockDim.x) {
        Ub[i + (int64_t)rank * l] = (float)(W[i + (int64_t)j * l] * inv);
        Vb[i + (int64_t)rank * l] = (float)V[i + (int64_t)j * l];
    }
}

// ------------------------------------------------------------------ launchers
cudaError_t launch_cast_rows(const float* src, int64_t lds, int64_t rows, int cols, const float* rscale, uint16_t* hi,
                             uint16_t* lo, int64_t ldd, int bf16, cudaStream_t st) {
    const int64_t total = rows * cols;
    RG_LAUNCH((cast_rows_kernel<float>), (unsigned)std::min<int64_t>((total + 255) / 256, 148 * 16), 256, 0, st, 
        src, lds, rows, cols, rscale, hi, lo, ldd, bf16);
    return cudaGetLastError();
}
cudaError_t launch_cast_rows64(const double* src, int64_t lds, int64_t rows, int cols, const float* rscale,
                               uint16_t* hi, uint16_t* lo, int64_t ldd, int bf16, cudaStream_t st) {
    const int64_t total = rows * cols;
    RG_LAUNCH((cast_rows_kernel<double>), (unsigned)std::min<int64_t>((total + 255) / 256, 148 * 16), 256, 0, st, 
        src, lds, rows, cols, rscale, hi, lo, ldd, bf16);
    return cudaGetLastError();
}

cudaError_t launch_unscale_rows(float* X, int64_t ldx, int64_t rows, int cols, const float* rscale, cudaStream_t st) {
    const int64_t total = rows * cols;
    RG_LAUNCH((unscale_rows_kernel), (unsigned)std::min<int64_t>((total + 255) / 256, 148 * 16), 256, 0, st, X, ldx, rows, cols,
                                                                                                      rscale);
    return cudaGetLastError();
}

cudaError_t launch_jacobi_svd(const float* R, int64_t ldr, int l, int r, double* W, double* V, double* sig, int* flags,
                              float* S, float* Ub, float* Vb, cudaStream_t st) {
    RG_LAUNCH((jacobi_init_kernel), (unsigned)std::min<int64_t>(((int64_t)l * l + 255) / 256, 148 * 8), 256, 0, st, R, ldr, l,
                                                                                                             W, V);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    int dev = 0, sms = 148, per_sm = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, jacobi_sweeps_kernel, 256, 0);
    int grid = std::min(sms * std::max(per_sm, 1), (l / 2 + 7) / 8 + 1);
    if (grid < 1) grid = 1;
    int max_sweeps = 40;
    double tol = 1e-13;
    void* args[] = {&W, &V, &l, &max_sweeps, &tol, &flags};
    ++g_launches;
    e = cudaLaunchCooperativeKernel((const void*)jacobi_sweeps_kernel, grid, 256, args, 0, st);
    if (e != cudaSuccess) return e;
    RG_LAUNCH((jacobi_extract_kernel), l, 256, 0, st, W, V, l, r, S, Ub, Vb, sig);
    e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    RG_LAUNCH((jacobi_rank_kernel), l, 256, 0, st, W, V, l, r, sig, S, Ub, Vb);
    return cudaGetLastError();
}

}  // namespace rg
