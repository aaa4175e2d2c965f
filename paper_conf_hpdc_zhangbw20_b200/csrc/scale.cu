// scale.cu -- column scaling of section 3.5 and the fused
// scale + fp32 copy + 16-bit cast that prepares the working matrix for Algorithm 1.
//
// AP = Q (R P): scaling the columns of A by a diagonal P leaves Q unchanged and scales
// the columns of R.  Reading #4: s_j = 2^(8 - floor(log2 ||a_j||_2)),
// i.e. every scaled column norm lies in [256, 512), so every fp16 operand of the
// recursion (|q| <= 1, |a2_ij| <= ||a_j||, |r_ij| <= ||a_j||) stays far below 65504, and
// powers of two make the scaling and the final unscaling R <- R P^{-1} exact.
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>

#include "kernels.h"

namespace rg {

constexpr int kNormChunk = 32768;     // rows per CTA of the column-norm pass
constexpr int kNormChunkMin = 2048;   // ... at most this short (narrow column ranges)

__device__ __forceinline__ uint16_t s_to16(float x, int bf16) {
    if (bf16) {
        __nv_bfloat16 b = __float2bfloat16_rn(x);
        return *reinterpret_cast<uint16_t*>(&b);
    }
    __half h = __float2half_rn(x);
    return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float s_from16(uint16_t u, int bf16) {
    if (bf16) return __bfloat162float(*reinterpret_cast<__nv_bfloat16*>(&u));
    return __half2float(*reinterpret_cast<__half*>(&u));
}

// partial[y * n + j] = sum_{i in chunk y} A(i, j)^2   (fp64 accumulation)
__global__ void __launch_bounds__(256) colnorm_partial_kernel(const float* __restrict__ A, int64_t lda, int64_t m,
                                                              int n, double* __restrict__ partial, int rows_per) {
    RG_PDL_ENTRY();
    const int j = blockIdx.x;
    const int64_t i0 = (int64_t)blockIdx.y * rows_per;
    const int64_t i1 = min(m, i0 + rows_per);
    const float* a = A + (int64_t)j * lda;
    double s = 0.0;
    const bool vec = ((reinterpret_cast<uintptr_t>(a + i0) & 15) == 0);
    if (vec) {
        const int64_t nv = (i1 - i0) / 4;
        const float4* a4 = reinterpret_cast<const float4*>(a + i0);
        for (int64_t v = threadIdx.x; v < nv; v += blockDim.x) {
            const float4 x = __ldg(a4 + v);
            s += (double)x.x * x.x + (double)x.y * x.y + (double)x.z * x.z + (double)x.w * x.w;
        }
        for (int64_t i = i0 + nv * 4 + threadIdx.x; i < i1; i += blockDim.x) s += (double)a[i] * a[i];
    } else {
        for (int64_t i = i0 + threadIdx.x; i < i1; i += blockDim.x) s += (double)a[i] * a[i];
    }
    __shared__ double red[8];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += red[w];
        partial[(int64_t)blockIdx.y * n + j] = t;
    }
}

// norm2[j] = sum_y partial (fixed order, deterministic).
__global__ void colnorm_sum_kernel(const double* __restrict__ partial, int chunks, int n, double* __restrict__ norm2) {
    RG_PDL_ENTRY();
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= n) return;
    double s = 0.0;
    for (int y = 0; y < chunks; ++y) s += partial[(int64_t)y * n + j];
    norm2[j] = s;
}

// scale[j] = power of two from the (global) squared column norm (reading #4), 1 if scaling
// is off; status[1] <- min column with a non-finite norm, status[0] <- min zero column.
__global__ void colscale_kernel(const double* __restrict__ norm2, int n, int do_scale, float* __restrict__ scale,
                                int* status, int col0) {
    RG_PDL_ENTRY();
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= n) return;
    const double s = norm2[j];
    if (!isfinite(s)) atomicMin(&status[1], col0 + j);
    else if (!(s > 0.0)) atomicMin(&status[0], col0 + j);
    float f = 1.0f;
    if (do_scale && s > 0.0 && isfinite(s)) {
        int e;
        frexp(sqrt(s), &e);              // ||a_j|| = frac * 2^e, frac in [0.5, 1)
        // scaled norm in [256, 512); the exponent is clamped to normal fp32 powers of two
        // (2^-126 .. 2^127) so the scale stays exact and finite: a column with a norm below
        // 2^-118 or above 2^135 is scaled as far as an exact power of two allows (a finite fp32
        // column norm is below 2^136, so only the tiny end can be left short of the target)
        const int ex = min(127, max(-126, 9 - e));
        f = ldexpf(1.0f, ex);
    }
    scale[j] = f;
}

// Q(:, j) = A(:, j) * scale[j] (fp32), Qh = 16-bit(Q), Ql = 16-bit((Q - Qh) 2^11) if non-null.
__global__ void __launch_bounds__(256) scale_cast_kernel(const float* __restrict__ A, int64_t lda, float* Q,
                                                         int64_t ldq, uint16_t* __restrict__ Qh,
                                                         uint16_t* __restrict__ Ql, int64_t ldh, int64_t m, int n,
                                                         const float* __restrict__ scale, int bf16) {
    RG_PDL_ENTRY();
    const int j = blockIdx.y;
    const float s = scale ? scale[j] : 1.0f;
    const float* a = A + (int64_t)j * lda;
    float* q = Q ? Q + (int64_t)j * ldq : nullptr;
    uint16_t* qh = Qh ? Qh + (int64_t)j * ldh : nullptr;
    uint16_t* ql = Ql ? Ql + (int64_t)j * ldh : nullptr;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const bool vec = ((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(q)) & 15) == 0 &&
                     (!qh || (reinterpret_cast<uintptr_t>(qh) & 7) == 0) &&
                     (!ql || (reinterpret_cast<uintptr_t>(ql) & 7) == 0);
    if (vec) {
        const int64_t nv = m / 4;
        for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < nv; v += stride) {
            float4 x = reinterpret_cast<const float4*>(a)[v];
            x.x *= s; x.y *= s; x.z *= s; x.w *= s;
            if (q) reinterpret_cast<float4*>(q)[v] = x;
            if (qh) {
                ushort4 h;
                h.x = s_to16(x.x, bf16); h.y = s_to16(x.y, bf16); h.z = s_to16(x.z, bf16); h.w = s_to16(x.w, bf16);
                reinterpret_cast<ushort4*>(qh)[v] = h;
                if (ql) {
                    ushort4 l;
                    l.x = s_to16((x.x - s_from16(h.x, bf16)) * 2048.f, bf16);
                    l.y = s_to16((x.y - s_from16(h.y, bf16)) * 2048.f, bf16);
                    l.z = s_to16((x.z - s_from16(h.z, bf16)) * 2048.f, bf16);
                    l.w = s_to16((x.w - s_from16(h.w, bf16)) * 2048.f, bf16);
                    reinterpret_cast<ushort4*>(ql)[v] = l;
                }
            }
        }
        for (int64_t i = nv * 4 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += stride) {
            const float x = a[i] * s;
            if (q) q[i] = x;
            if (qh) {
                const uint16_t h = s_to16(x, bf16);
                qh[i] = h;
                if (ql) ql[i] = s_to16((x - s_from16(h, bf16)) * 2048.f, bf16);
            }
        }
    } else {
        for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += stride) {
            const float x = a[i] * s;
            if (q) q[i] = x;
            if (qh) {
                const uint16_t h = s_to16(x, bf16);
                qh[i] = h;
                if (ql) ql[i] = s_to16((x - s_from16(h, bf16)) * 2048.f, bf16);
            }
        }
    }
}

// R(:, j) <- R(:, j) / scale[j] (exact: powers of two) for j in [c0, c0 + nc); strictly-lower
// part zeroed.  grid.y walks the columns, grid.x x 256 threads the rows (coalesced, no division).
__global__ void __launch_bounds__(256) unscale_r_kernel(float* R, int64_t ldr, int n, const float* __restrict__ scale,
                                                        int c0, int nc) {
    RG_PDL_ENTRY();
    for (int jj = blockIdx.y; jj < nc; jj += gridDim.y) {
        const int j = c0 + jj;
        const float s = scale ? scale[j] : 1.0f;
        float* r = R + (int64_t)j * ldr;
        for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
            r[i] = (i <= j) ? (scale ? r[i] / s : r[i]) : 0.f;
    }
}

cudaError_t launch_colnorm(const float* A, int64_t lda, int64_t m, int n, double* partial, double* norm2,
                           cudaStream_t st) {
    // kNormChunk rows per CTA; narrow column ranges (the chunked scaling pass) use shorter row
    // chunks (down to kNormChunkMin) so that the grid still covers ~8 CTAs per SM
    int rows_per = kNormChunk;
    while (rows_per > kNormChunkMin && (int64_t)n * ((m + rows_per - 1) / rows_per) < 148 * 8) rows_per >>= 1;
    const int chunks = (int)((m + rows_per - 1) / rows_per);
    dim3 grid(n, chunks);
    RG_LAUNCH((colnorm_partial_kernel), grid, 256, 0, st, A, lda, m, n, partial, rows_per);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    RG_LAUNCH((colnorm_sum_kernel), (n + 127) / 128, 128, 0, st, partial, chunks, n, norm2);
    return cudaGetLastError();
}

cudaError_t launch_colscale(const double* norm2, int n, int do_scale, float* scale, int* status, int col0,
                            cudaStream_t st) {
    RG_LAUNCH((colscale_kernel), (n + 127) / 128, 128, 0, st, norm2, n, do_scale, scale, status, col0);
    return cudaGetLastError();
}

size_t colnorm_partial_doubles(int64_t m, int n) {
    return (size_t)((m + kNormChunkMin - 1) / kNormChunkMin) * (size_t)n;
}

cudaError_t launch_scale_cast(const float* A, int64_t lda, float* Q, int64_t ldq, uint16_t* Qh, uint16_t* Ql,
                              int64_t ldh, int64_t m, int n, const float* scale, int bf16, cudaStream_t st) {
    // ~8 waves of 256-thread CTAs over the whole matrix, split over columns (grid.y)
    int64_t per_col = (m / 4 + 255) / 256;
    int64_t target = (148LL * 8 * 8 + n - 1) / n;
    int bx = (int)(per_col < target ? per_col : target);
    if (bx < 1) bx = 1;
    dim3 grid(bx, n);
    RG_LAUNCH((scale_cast_kernel), grid, 256, 0, st, A, lda, Q, ldq, Qh, Ql, ldh, m, n, scale, bf16);
    return cudaGetLastError();
}

cudaError_t launch_unscale_r(float* R, int64_t ldr, int n, const float* scale, cudaStream_t st, int c0, int nc) {
    if (nc < 0) nc = n - c0;
    if (nc <= 0 || n <= 0) return cudaSuccess;
    const int bx = (n + 255) / 256 < 4 ? (n + 255) / 256 : 4;
    const int by = nc < 65535 ? nc : 65535;
    RG_LAUNCH((unscale_r_kernel), dim3(bx, by), 256, 0, st, R, ldr, n, scale, c0, nc);
    return cudaGetLastError();
}

}  // namespace rg
