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
#include <cstdio>
#include <cstdlib>

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
                                   double* __restrict__ V, int trans) {
    RG_PDL_ENTRY();
    const int64_t total = (int64_t)l * l;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int i = (int)(e % l), j = (int)(e / l);
        if (trans)
            W[e] = (j <= i) ? (double)R[j + (int64_t)i * ldr] : 0.0;
        else
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

// ------------------------------------------------------------------ cluster Jacobi (l <= 544)
// Same rotations, block-cyclic parallel ordering, columns resident in registers.  A thread-block
// cluster of cs CTAs x wper warps covers 2 cs wper >= l columns (padding columns are zero and never
// rotated); warp i of a CTA holds one column of each of the CTA's two blocks (x: "top" block,
// y: "bot" block), NPL doubles per lane (element u * 32 + lane).  One sweep:
//   1. all pairs among the CTA's own 2 wper columns: round-robin (Brent-Luk) over its warps, column
//      moves through shared memory (the two blocks are then re-formed as the x-set and y-set);
//   2. 2 cs - 2 rounds of a round-robin over the 2 cs blocks between CTAs (block moves by
//      distributed-shared-memory stores, two cluster barriers per round); in each, the wper x wper
//      pairs of the CTA's two blocks: wper local rounds, the y block shifted one warp per round.
// Every pair of columns meets once per sweep (intra-block pairs in step 1, the CTA's own block pair
// in step 1, every other block pair in step 2).  Converged when no rotation fired in a sweep.
// V is not accumulated: V_b = R^T W S^{-2} afterwards (jacobi_rank_rt_kernel).  At l = 528 this
// replaces a one-pair-per-warp ordering with 527 cluster-synchronised rounds per sweep (28 ms) and
// a grid-synchronised kernel with L2-latency-bound rounds (70 ms).
// Cluster barrier with cluster-scope release/acquire (orders the DSMEM column stores before the
// receivers' loads).  cooperative_groups' cluster.sync() emitted a GPU-scope MEMBAR per call.
__device__ __forceinline__ void jc_cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

template <int NPL>
__device__ __forceinline__ double jc_dot(const double (&x)[NPL], const double (&y)[NPL]) {
    double g0 = 0.0, g1 = 0.0;   // two accumulators: halves the dependent DFMA chain
#pragma unroll
    for (int u = 0; u < NPL; u += 2) {
        g0 = fma(x[u], y[u], g0);
        if (u + 1 < NPL) g1 = fma(x[u + 1], y[u + 1], g1);
    }
    return wsum(g0 + g1);
}

// One Hestenes rotation of (x, y) with their squared norms a, b carried along (updated as
// a - t g, b + t g instead of recomputed: one dot product per rotation).
template <int NPL>
__device__ __forceinline__ bool jc_rotate(double (&x)[NPL], double (&y)[NPL], double& a, double& b, int ix, int iy,
                                          int l, double tol) {
    if (ix >= l || iy >= l) return false;
    const double g = jc_dot<NPL>(x, y);
    if (g * g <= tol * tol * (a * b) || g == 0.0) return false;
    const double zeta = (b - a) / (2.0 * g);
    const double t = (zeta >= 0.0 ? 1.0 : -1.0) / (fabs(zeta) + sqrt(1.0 + zeta * zeta));
    const double c = rsqrt(1.0 + t * t), sn = c * t;
#pragma unroll
    for (int u = 0; u < NPL; ++u) {
        const double xv = x[u], yv = y[u];
        x[u] = c * xv - sn * yv;
        y[u] = sn * xv + c * yv;
    }
    a -= t * g;
    b += t * g;
    return true;
}

// Rotation angle from (a, b, g) = (|x|^2, |y|^2, x^T y); false when the pair is already
// orthogonal to tol (or involves a padding column).
// fp64 reciprocal / reciprocal square root: hardware approximation (MUFU, ~2^-23) + Newton
// steps.  The rotation's dependent chain is latency-bound (one rotation per warp per round), and
// the IEEE div / sqrt sequences dominated it.  t only steers convergence; c is refined to ~2^-50 so
// that c^2 (1 + t^2) = 1 keeps the column norms (the singular values) intact.
__device__ __forceinline__ double jc_rcp(double x) {
    double y;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    double e = fma(-x, y, 1.0);
    y = fma(y, e, y);
    e = fma(-x, y, 1.0);
    return fma(y, e, y);
}
__device__ __forceinline__ double jc_rsqrt(double x) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    y = y * fma(-0.5 * x * y, y, 1.5);
    return y * fma(-0.5 * x * y, y, 1.5);
}
__device__ __forceinline__ bool jc_angle(double a, double b, double g, double tol, double& c, double& sn, double& t) {
    if (g * g <= tol * tol * (a * b) || g == 0.0) return false;
    const double zeta = (b - a) * jc_rcp(2.0 * g);
    const double az = fabs(zeta);
    const double q = 1.0 + zeta * zeta;
    const double sq = q * jc_rsqrt(q);   // sqrt(1 + zeta^2)
    t = (zeta >= 0.0 ? 1.0 : -1.0) * jc_rcp(az + sq);
    c = jc_rsqrt(1.0 + t * t);
    sn = c * t;
    return true;
}

// Rotation of the register column x (squared norm a) with the shared-memory column yc (norm *nb).
// y is streamed from shared memory twice (dot, then update) instead of held in registers: the
// 17-warp CTAs of l = 528 have 96 registers per thread.
template <int NPL>
__device__ __forceinline__ bool jc_rotate_smem(double (&x)[NPL], double& a, int ix, double* yc, double* nb, int iy,
                                               int l, double tol, int lane) {
    if (ix >= l || iy >= l) return false;
    double g0 = 0.0, g1 = 0.0;
#pragma unroll
    for (int u = 0; u < NPL; u += 2) {
        g0 = fma(x[u], yc[u * 32 + lane], g0);
        if (u + 1 < NPL) g1 = fma(x[u + 1], yc[(u + 1) * 32 + lane], g1);
    }
    const double g = wsum(g0 + g1);
    const double b = *nb;
    double c, sn, t;
    if (!jc_angle(a, b, g, tol, c, sn, t)) return false;
#pragma unroll
    for (int u = 0; u < NPL; ++u) {
        const double xv = x[u], yv = yc[u * 32 + lane];
        x[u] = c * xv - sn * yv;
        yc[u * 32 + lane] = sn * xv + c * yv;
    }
    a -= t * g;
    __syncwarp();
    if (lane == 0) *nb = b + t * g;
    return true;
}

// Rotation of two shared-memory columns (norms *na, *nb), streamed.
template <int NPL>
__device__ __forceinline__ bool jc_rotate_2smem(double* xc, double* na, int ix, double* yc, double* nb, int iy, int l,
                                                double tol, int lane) {
    if (ix >= l || iy >= l) return false;
    double g0 = 0.0, g1 = 0.0;
#pragma unroll
    for (int u = 0; u < NPL; u += 2) {
        g0 = fma(xc[u * 32 + lane], yc[u * 32 + lane], g0);
        if (u + 1 < NPL) g1 = fma(xc[(u + 1) * 32 + lane], yc[(u + 1) * 32 + lane], g1);
    }
    const double g = wsum(g0 + g1);
    const double a = *na, b = *nb;
    double c, sn, t;
    if (!jc_angle(a, b, g, tol, c, sn, t)) return false;
#pragma unroll
    for (int u = 0; u < NPL; ++u) {
        const double xv = xc[u * 32 + lane], yv = yc[u * 32 + lane];
        xc[u * 32 + lane] = c * xv - sn * yv;
        yc[u * 32 + lane] = sn * xv + c * yv;
    }
    __syncwarp();
    if (lane == 0) {
        *na = a - t * g;
        *nb = b + t * g;
    }
    return true;
}

template <int NPL>
__global__ void __launch_bounds__(544, 1) jacobi_cluster_kernel(double* __restrict__ W, int l, int wper,
                                                                int max_sweeps, double tol, int* flags) {
    cg::cluster_group cl = cg::this_cluster();
    extern __shared__ __align__(16) double jc_smem[];
    // slots 0 .. wper - 1: the x block, wper .. 2 wper - 1: the y block (NPL * 32 doubles each)
    double* buf = jc_smem;
    double* snrm = buf + (size_t)2 * wper * NPL * 32;   // [2 wper] squared norms
    int* sid = reinterpret_cast<int*>(snrm + 2 * wper); // [2 wper] column ids
    __shared__ int rot_flag;
    const int crank = (int)cl.block_rank();
    const int cs = (int)cl.num_blocks();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    auto col = [&](int slot) { return buf + (size_t)slot * NPL * 32; };
    // x (this warp's column of the x block) in registers; the y block in shared memory
    double x[NPL];
    int ix = (2 * crank) * wper + warp;
    double na = 0.0;
    {
        const int iy = (2 * crank + 1) * wper + warp;
        double* yc = col(wper + warp);
#pragma unroll
        for (int u = 0; u < NPL; ++u) {
            const int i = u * 32 + lane;
            x[u] = (ix < l && i < l) ? W[(int64_t)ix * l + i] : 0.0;
            yc[u * 32 + lane] = (iy < l && i < l) ? W[(int64_t)iy * l + i] : 0.0;
        }
        if (lane == 0) sid[wper + warp] = iy;
    }
    int sweep = 0;
    for (; sweep < max_sweeps; ++sweep) {
        if (threadIdx.x == 0) rot_flag = 0;
        bool any = false;
        // ---- 1. all pairs among the CTA's 2 wper columns: x block to shared memory, circle-method
        // round robin over the 2 wper slots (pairs of slots, no column moves)
        {
            double* xc = col(warp);
#pragma unroll
            for (int u = 0; u < NPL; ++u) xc[u * 32 + lane] = x[u];
            double yy = 0.0;
            const double* yc = col(wper + warp);
#pragma unroll
            for (int u = 0; u < NPL; ++u) yy = fma(yc[u * 32 + lane], yc[u * 32 + lane], yy);
            yy = wsum(yy);
            na = jc_dot<NPL>(x, x);   // exact norms once per sweep (rotations update them)
            if (lane == 0) {
                sid[warp] = ix;
                snrm[warp] = na;
                snrm[wper + warp] = yy;
            }
        }
        __syncthreads();
        for (int r = 0; r < 2 * wper - 1; ++r) {
            int p, q;
            rr_pair(2 * wper, r, warp, p, q);
            any |= jc_rotate_2smem<NPL>(col(p), snrm + p, sid[p], col(q), snrm + q, sid[q], l, tol, lane);
            __syncthreads();
        }
        {
            const double* xc = col(warp);
#pragma unroll
            for (int u = 0; u < NPL; ++u) x[u] = xc[u * 32 + lane];
            na = snrm[warp];
        }
        // ---- 2. block pairs between CTAs (pull form of the block round robin):
        //   new x(c) = x(0) (c = 0), y(0) (c = 1), x(c - 1);   new y(c) = y(c + 1), x(cs - 1) (c = cs - 1)
        for (int tr = 1; tr <= 2 * cs - 2; ++tr) {
            {
                double* xc = col(warp);
#pragma unroll
                for (int u = 0; u < NPL; ++u) xc[u * 32 + lane] = x[u];
                if (lane == 0) {
                    sid[warp] = ix;
                    snrm[warp] = na;
                }
            }
            jc_cluster_sync();
            double ny[NPL];
            int iny;
            double nny;
            {
                const int src_c = crank == cs - 1 ? crank : crank + 1;
                const int src_s = crank == cs - 1 ? warp : wper + warp;
                const double* ycr = cl.map_shared_rank(col(src_s), src_c);
#pragma unroll
                for (int u = 0; u < NPL; ++u) ny[u] = ycr[u * 32 + lane];
                iny = *cl.map_shared_rank(sid + src_s, src_c);
                nny = *cl.map_shared_rank(snrm + src_s, src_c);
            }
            if (crank >= 1) {
                const int src_c = crank - 1;
                const int src_s = crank == 1 ? wper + warp : warp;
                const double* xcr = cl.map_shared_rank(col(src_s), src_c);
#pragma unroll
                for (int u = 0; u < NPL; ++u) x[u] = xcr[u * 32 + lane];
                ix = *cl.map_shared_rank(sid + src_s, src_c);
                na = *cl.map_shared_rank(snrm + src_s, src_c);
            }
            jc_cluster_sync();
            {
                double* yc = col(wper + warp);
#pragma unroll
                for (int u = 0; u < NPL; ++u) yc[u * 32 + lane] = ny[u];
                if (lane == 0) {
                    sid[wper + warp] = iny;
                    snrm[wper + warp] = nny;
                }
            }
            __syncthreads();
            // the wper x wper pairs (x_i, y_{(i + s) mod wper})
            for (int sft = 0; sft < wper; ++sft) {
                const int ys = wper + (warp + sft) % wper;
                any |= jc_rotate_smem<NPL>(x, na, ix, col(ys), snrm + ys, sid[ys], l, tol, lane);
                __syncthreads();
            }
        }
        if (any && lane == 0) atomicOr(&rot_flag, 1);
        jc_cluster_sync();
        int tot = 0;
        for (int c = 0; c < cs; ++c) tot |= *cl.map_shared_rank(&rot_flag, c);
        jc_cluster_sync();
        if (!tot) {
            ++sweep;
            break;
        }
    }
    {
        const double* yc = col(wper + warp);
        const int iy = sid[wper + warp];
#pragma unroll
        for (int u = 0; u < NPL; ++u) {
            const int i = u * 32 + lane;
            if (i < l) {
                if (ix < l) W[(int64_t)ix * l + i] = x[u];
                if (iy < l) W[(int64_t)iy * l + i] = yc[u * 32 + lane];
            }
        }
    }
    if (crank == 0 && threadIdx.x == 0) flags[1] = sweep;
}

// Ranks by descending sigma_j = |w_j| (ties by index); for rank < r: S, Ub(:, rank) = w_j / sigma_j,
// Vb(:, rank) = R^T w_j / sigma_j^2 (R = U_b S V_b^T => V_b = R^T U_b S^{-1}); fp64, one CTA per j.
__global__ void jacobi_rank_rt_kernel(const double* __restrict__ W, const float* __restrict__ R, int64_t ldr, int l,
                                      int r, const double* __restrict__ sig, float* __restrict__ S,
                                      float* __restrict__ Ub, float* __restrict__ Vb, int trans) {
    RG_PDL_ENTRY();
    extern __shared__ double wcol[];
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
    for (int i = threadIdx.x; i < l; i += blockDim.x) wcol[i] = W[i + (int64_t)j * l];
    __syncthreads();
    const int rank = s_rank;
    if (rank >= r) return;
    const double sj = sig[j];
    if (threadIdx.x == 0) S[rank] = (float)sj;
    const double inv = sj > 0.0 ? 1.0 / sj : 0.0;
    // trans = 0: W = R J = U_b S, V_b = R^T W S^-2.  trans = 1: W = R^T J = V_b S, U_b = R W S^-2.
    float* Wout = trans ? Vb : Ub;
    float* Oout = trans ? Ub : Vb;
    for (int i = threadIdx.x; i < l; i += blockDim.x) {
        Wout[i + (int64_t)rank * l] = (float)(wcol[i] * inv);
        double v = 0.0;
        if (trans) {
            for (int k = i; k < l; ++k) v = fma((double)R[i + (int64_t)k * ldr], wcol[k], v);   // row i of R
        } else {
            const float* rc = R + (int64_t)i * ldr;   // column i of R: R(k, i), k <= i
            for (int k = 0; k <= i; ++k) v = fma((double)rc[k], wcol[k], v);
        }
        Oout[i + (int64_t)rank * l] = (float)(v * inv * inv);
    }
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

size_t jacobi_w_doubles(int l) { return (size_t)l * std::max(l, svd_bj_cols(l)); }

cudaError_t launch_jacobi_svd(const float* R, int64_t ldr, int l, int r, double* W, double* V, double* sig, int* flags,
                              float* S, float* Ub, float* Vb, cudaStream_t st) {
    if (svd_bj_fits(l) && getenv("RGSQR_JACOBI_GRID") == nullptr && getenv("RGSQR_JACOBI_CLUSTER") == nullptr) {
        // block one-sided Jacobi (svd.cu) on W = R^T (reading #22): W -> V_R S, U_R = R W S^-2
        RG_LAUNCH((jacobi_init_kernel), (unsigned)std::min<int64_t>(((int64_t)l * l + 255) / 256, 148 * 8), 256, 0, st,
                  R, ldr, l, W, V, 1);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        const int cols = svd_bj_cols(l);
        if (cols > l) {
            e = cudaMemsetAsync(W + (size_t)l * l, 0, (size_t)l * (cols - l) * 8, st);
            if (e != cudaSuccess) return e;
        }
        const double jtol = getenv("RGSQR_JACOBI_TOL") ? atof(getenv("RGSQR_JACOBI_TOL")) : 1e-12;
        int sweeps = 0;
        e = launch_svd_bj(W, l, 30, jtol, reinterpret_cast<unsigned long long*>(flags + 2), &sweeps, st);
        if (e != cudaSuccess) return e;
        if (getenv("RGSQR_JACOBI_TRACE")) fprintf(stderr, "[rgsqr svd] block Jacobi l = %d: %d sweeps\n", l, sweeps);
        RG_LAUNCH((jacobi_extract_kernel), l, 256, 0, st, W, V, l, r, S, Ub, Vb, sig);
        e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        RG_LAUNCH((jacobi_rank_rt_kernel), l, 256, (size_t)l * 8, st, W, R, ldr, l, r, sig, S, Ub, Vb, 1);
        return cudaGetLastError();
    }
    const bool cluster = l <= 544 && getenv("RGSQR_JACOBI_GRID") == nullptr;
    // one-sided Jacobi on R^T (the graded, lower-triangular transpose) needs about half the sweeps
    // of Jacobi on R (measured 11 vs 21 at l = 528)
    const int trans = cluster ? (getenv("RGSQR_JACOBI_T") != nullptr ? atoi(getenv("RGSQR_JACOBI_T")) : 1) : 0;
    const double jtol = getenv("RGSQR_JACOBI_TOL") ? atof(getenv("RGSQR_JACOBI_TOL")) : 1e-13;
    RG_LAUNCH((jacobi_init_kernel), (unsigned)std::min<int64_t>(((int64_t)l * l + 255) / 256, 148 * 8), 256, 0, st, R, ldr, l,
                                                                                                             W, V, trans);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    if (cluster) {
        // 2 cs wper >= l columns, <= 17 warps (544 threads) per CTA, <= 16 CTAs per cluster
        const int P = (l + 1) / 2;
        const int cs = std::max(1, std::min(16, (P + 16) / 17));
        const int wper = (P + cs - 1) / cs;
        const int npl = (l + 31) / 32;
        int max_sweeps = 40;
        double tol = jtol;
        cudaLaunchConfig_t cfg{};
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = cs;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.gridDim = dim3(cs);
        cfg.blockDim = dim3(32 * wper);
        cfg.stream = st;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        auto go = [&](auto kern, int np) -> cudaError_t {
            cfg.dynamicSmemBytes = (size_t)2 * wper * np * 32 * 8 + (size_t)wper * 2 * (8 + 4) + 16;   // x + y blocks
            cudaError_t e2 = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                  (int)cfg.dynamicSmemBytes);
            if (e2 != cudaSuccess) return e2;
            if (cs > 8) {
                e2 = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
                if (e2 != cudaSuccess) return e2;
            }
            ++g_launches;
            return cudaLaunchKernelEx(&cfg, kern, W, l, wper, max_sweeps, tol, flags);
        };
        if (npl <= 4) e = go(jacobi_cluster_kernel<4>, 4);
        else if (npl <= 8) e = go(jacobi_cluster_kernel<8>, 8);
        else if (npl <= 12) e = go(jacobi_cluster_kernel<12>, 12);
        else e = go(jacobi_cluster_kernel<17>, 17);
        if (e != cudaSuccess) return e;
        RG_LAUNCH((jacobi_extract_kernel), l, 256, 0, st, W, V, l, r, S, Ub, Vb, sig);
        e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        RG_LAUNCH((jacobi_rank_rt_kernel), l, 256, (size_t)l * 8, st, W, R, ldr, l, r, sig, S, Ub, Vb, trans);
        return cudaGetLastError();
    }
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
