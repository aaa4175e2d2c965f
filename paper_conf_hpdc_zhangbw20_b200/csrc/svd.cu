// svd.cu -- block one-sided Jacobi SVD (fp64) of the small l x l triangular factors of
// lowrank_approx (R_b, section 3.4 / config 5) and lowrank_qrsvd (R, section 3.4 / Table 4).
//
// One-sided Jacobi (Hestenes) orthogonalises the columns of W (= R^T, reading #22) by plane
// rotations; here the columns are grouped into blocks of 16 and a round-robin tournament pairs
// blocks (I, J).  For a pair, the 32 columns W_IJ = [W_I W_J] are orthogonalised as a unit:
//   M = W_IJ^T W_IJ (32 x 32 Gram, fp64),  U = one cyclic Jacobi sweep on M (the standard
//   "block Jacobi with one inner sweep"),  W_IJ <- W_IJ U.
// A sweep is nblk - 1 rounds; converged when every pair's Gram has max |M_ij| / sqrt(M_ii M_jj)
// < tol at the start of a sweep.  The column norms of the converged W are the singular values.
//
// B200 mapping: one round = one launch; a pair = a thread-block cluster of C CTAs splitting the
// l rows (32 pairs x 4 = 128 CTAs at l = 1024).  Per CTA: its rows of W_IJ in
// shared memory, the partial Gram on the fp64 tensor cores (DMMA m8n8k4, one fragment per 8-column
// block serves as A and B), a deterministic cluster all-reduce through distributed shared memory
// (reduce-scatter in rank order + all-gather), the 32 x 32 inner sweep done redundantly by every
// CTA of the cluster (identical inputs -> identical U, no broadcast), the update W_IJ U on DMMA
// (each warp owns 8 rows, so it overwrites only what it read), and the store.  The scalar
// tournament of lowrank.cu needed one grid-wide step per column pair round (1023 per sweep at
// l = 1024); here a sweep is 63 launches.  (64-column pairs measured 254 us per round: the two-sided
// 64 x 64 inner sweep is shared-memory-bandwidth bound, 128 KB of M / U traffic per inner round.)
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstdio>
#include <cstring>

#include "kernels.h"

namespace cg = cooperative_groups;

namespace rg {

constexpr int BJ_B = 16;                 // columns per block
constexpr int BJ_W = 2 * BJ_B;           // 32 columns per pair
constexpr int BJ_THREADS = 512;
constexpr int BJ_NW = BJ_THREADS / 32;
constexpr int BJ_MLD = BJ_W + 1;         // inner M row stride (doubles)
constexpr int BJ_ULD = BJ_W + 4;         // inner U row stride (doubles)
constexpr int BJ_NE = BJ_W * (BJ_W + 1) / 2;   // packed upper Gram entries
constexpr int BJ_MAX_ROWS = 320;         // rows per CTA
constexpr int BJ_NB8 = BJ_W / 8;         // 8-column blocks of a pair
constexpr int BJ_NT = BJ_NB8 * (BJ_NB8 + 1) / 2;   // upper 8 x 8 Gram blocks (10)
constexpr int BJ_GROUPS = 2;             // Gram warps = groups (BJ_NT / BJ_GROUPS blocks each) x k-slices
constexpr int BJ_TPG = BJ_NT / BJ_GROUPS;
constexpr int BJ_KS = BJ_NW / BJ_GROUPS; // 8 k-slices
static_assert(BJ_NT % BJ_GROUPS == 0, "Gram block groups");

struct BjArgs {
    double* W;            // l rows x (nblk * 32) columns, column-major, ld = l (padding columns zero)
    int l;
    int nblk;             // even
    int C;                // CTAs per pair (cluster size)
    int rpc;              // rows per CTA
    int lds;              // shared-memory column stride of the W tile (doubles, == 4 mod 16)
    int sweep, round;
    double tol;
    unsigned long long* maxoff;   // [sweep]: max off-diagonal ratio seen in that sweep (double bits)
};

__device__ __forceinline__ void bj_pair(int L, int r, int k, int& p, int& q) {   // round-robin tournament
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

__host__ __device__ constexpr int bj_blk_i(int t) {   // upper blocks row by row
    int bi = 0;
    while (t >= BJ_NB8 - bi) {
        t -= BJ_NB8 - bi;
        ++bi;
    }
    return bi;
}
__host__ __device__ constexpr int bj_blk_j(int t) {
    int bi = 0;
    while (t >= BJ_NB8 - bi) {
        t -= BJ_NB8 - bi;
        ++bi;
    }
    return bi + t;
}

__device__ __forceinline__ double bj_rcp(double d) {
    double y;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(d));
    const double e = fma(-d, y, 1.0);
    return fma(y, e, y);
}
__device__ __forceinline__ double bj_rsqrt(double d) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(d));
    const double e = fma(-d * y, y, 1.0);
    return fma(0.5 * y, e, y);
}

__device__ __forceinline__ void bj_dmma(double (&d)[2], double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(d[0]), "+d"(d[1])
                 : "d"(a), "d"(b));
}

template <int T>
__device__ __forceinline__ void bj_blk(double (&acc)[2], const double (&f)[BJ_NB8]) {
    constexpr int bi = bj_blk_i(T), bj = bj_blk_j(T);   // compile-time: f stays in registers
    bj_dmma(acc, f[bi], f[bj]);
}

template <int Q, int U>
struct BjGroup {   // blocks Q, Q + G, Q + 2G, ... of the group
    static __device__ __forceinline__ void run(double (&acc)[BJ_TPG][2], const double (&f)[BJ_NB8]) {
        bj_blk<Q + BJ_GROUPS * U>(acc[U], f);
        BjGroup<Q, U + 1>::run(acc, f);
    }
};
template <int Q>
struct BjGroup<Q, BJ_TPG> {
    static __device__ __forceinline__ void run(double (&)[BJ_TPG][2], const double (&)[BJ_NB8]) {}
};

template <int Q>
__device__ __forceinline__ void bj_gram_group(const double* Ws, int lds, int rows4, int ks, int lane,
                                              double (&acc)[BJ_TPG][2]) {
    const int g = lane >> 2, c = lane & 3;
    const double* col = Ws + g * lds + c;
#pragma unroll 1
    for (int k0 = 4 * ks; k0 < rows4; k0 += 4 * BJ_KS) {
        double f[BJ_NB8];
#pragma unroll
        for (int b = 0; b < BJ_NB8; ++b) f[b] = col[8 * b * lds + k0];
        BjGroup<Q, 0>::run(acc, f);
    }
}

__global__ void __launch_bounds__(BJ_THREADS, 1) svd_bj_round_kernel(BjArgs a) {
    cg::cluster_group cl = cg::this_cluster();
    if (a.sweep > 0) {
        const double prev = __longlong_as_double((long long)a.maxoff[a.sweep - 1]);
        if (prev < a.tol) return;   // uniform over the grid: converged in an earlier sweep
    }
    extern __shared__ __align__(16) double bj_smem[];
    double* Ws = bj_smem;                                   // BJ_W x lds
    double* part = Ws + BJ_W * a.lds;                       // packed partial Gram (BJ_NE)
    double* msum = part + BJ_NE;                            // packed reduced Gram (BJ_NE)
    double* M = msum + BJ_NE;                               // BJ_W x BJ_MLD
    double* U = M + BJ_W * BJ_MLD;                          // BJ_W x BJ_ULD (row-major)
    double* scr = U + BJ_W * BJ_ULD;                        // BJ_NT x 64 (k-slice exchange)
    __shared__ double s_a[BJ_W], s_b[BJ_W];
    __shared__ int s_o[BJ_W];
    __shared__ double s_off[BJ_NW];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int cr = (int)cl.block_rank();
    const int pair = blockIdx.x / a.C;
    int bI, bJ;
    bj_pair(a.nblk, a.round, pair, bI, bJ);
    const int r0 = cr * a.rpc;
    const int rows = max(0, min(a.rpc, a.l - r0));
    const int rows4 = (rows + 7) & ~7;   // whole 8-row DMMA blocks (zero rows beyond `rows`)
    // ---- 1. load this CTA's rows of the 64 columns (zero beyond)
    for (int e = tid; e < BJ_W * rows4; e += BJ_THREADS) {
        const int lc = e / rows4, i = e % rows4;
        const int gc = lc < BJ_B ? bI * BJ_B + lc : bJ * BJ_B + (lc - BJ_B);
        Ws[lc * a.lds + i] = (i < rows) ? a.W[(int64_t)gc * a.l + r0 + i] : 0.0;
    }
    __syncthreads();
    // ---- 2. partial Gram on DMMA: warp = group q (BJ_TPG of the upper 8x8 blocks) x k-slice ks
    {
        const int q = warp % BJ_GROUPS, ks = warp / BJ_GROUPS;
        double acc[BJ_TPG][2];
#pragma unroll
        for (int u = 0; u < BJ_TPG; ++u) acc[u][0] = acc[u][1] = 0.0;
        if (q == 0) bj_gram_group<0>(Ws, a.lds, rows4, ks, lane, acc);
        else bj_gram_group<1>(Ws, a.lds, rows4, ks, lane, acc);
        static_assert(BJ_GROUPS == 2, "group dispatch");
        constexpr int NENT = BJ_NT * 64;
        constexpr int NQ = (NENT + BJ_THREADS - 1) / BJ_THREADS;
        double run[NQ];
#pragma unroll
        for (int i = 0; i < NQ; ++i) run[i] = 0.0;
        for (int r = 0; r < BJ_KS; ++r) {   // the k-slices summed in order
            __syncthreads();
            if (ks == r) {
                double* dst = scr + q * BJ_TPG * 64 + lane;
#pragma unroll
                for (int u = 0; u < BJ_TPG; ++u) {
                    dst[(2 * u) * 32] = acc[u][0];
                    dst[(2 * u + 1) * 32] = acc[u][1];
                }
            }
            __syncthreads();
#pragma unroll
            for (int i = 0; i < NQ; ++i) {
                const int e = tid + BJ_THREADS * i;
                if (e < NENT) run[i] += scr[e];
            }
        }
#pragma unroll
        for (int i = 0; i < NQ; ++i) {
            const int e = tid + BJ_THREADS * i;
            if (e < NENT) {
                const int ln = e & 31, v = (e >> 5) & 1, qu = e >> 6, qq = qu / BJ_TPG, u = qu % BJ_TPG;
                const int t = qq + BJ_GROUPS * u;
                const int ii = 8 * bj_blk_i(t) + (ln >> 2), jj = 8 * bj_blk_j(t) + 2 * (ln & 3) + v;
                if (ii <= jj) part[jj * (jj + 1) / 2 + ii] = run[i];
            }
        }
    }
    // ---- 3. cluster all-reduce (fixed rank order): reduce-scatter, then all-gather
    cl.sync();
    const int slice = (BJ_NE + a.C - 1) / a.C;
    {
        const int e0 = cr * slice, e1 = min(BJ_NE, e0 + slice);
        for (int e = e0 + tid; e < e1; e += BJ_THREADS) {
            double s = 0.0;
            for (int r = 0; r < a.C; ++r) s += cl.map_shared_rank(part, r)[e];
            msum[e] = s;
        }
    }
    cl.sync();
    for (int r = 0; r < a.C; ++r) {
        if (r == cr) continue;
        const double* src = cl.map_shared_rank(msum, r);
        const int e0 = r * slice, e1 = min(BJ_NE, e0 + slice);
        for (int e = e0 + tid; e < e1; e += BJ_THREADS) msum[e] = src[e];
    }
    __syncthreads();
    // full symmetric M, U = I; convergence measure of this pair (before its rotations)
    double off = 0.0;
    for (int e = tid; e < BJ_W * BJ_W; e += BJ_THREADS) {
        const int i = e / BJ_W, j = e % BJ_W;
        const int lo = min(i, j), hi = max(i, j);
        M[i * BJ_MLD + j] = msum[hi * (hi + 1) / 2 + lo];
        U[i * BJ_ULD + j] = (i == j) ? 1.0 : 0.0;
        if (i < j) {
            const double d = msum[i * (i + 1) / 2 + i] * msum[j * (j + 1) / 2 + j];
            if (d > 0.0) off = fmax(off, fabs(msum[j * (j + 1) / 2 + i]) * rsqrt(d));
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) off = fmax(off, __shfl_xor_sync(0xffffffffu, off, o));
    if (lane == 0) s_off[warp] = off;
    __syncthreads();
    double pair_off = 0.0;
    for (int w = 0; w < BJ_NW; ++w) pair_off = fmax(pair_off, s_off[w]);
    if (tid == 0 && cr == 0) atomicMax(a.maxoff + a.sweep, (unsigned long long)__double_as_longlong(pair_off));
    // threshold Jacobi: a pair already orthogonal to the sweep tolerance is left as it is (every CTA
    // of the cluster reduced the same Gram, so the decision is uniform over the cluster)
    if (pair_off < a.tol) {
        cl.sync();   // no CTA leaves while a cluster peer may still read its shared memory
        return;
    }
    // ---- 4. one cyclic Jacobi sweep on M (64 indices, 63 rounds of 32 disjoint rotations);
    // every CTA of the cluster computes the same U
    for (int rr = 0; rr < BJ_W - 1; ++rr) {
        if (tid < BJ_W / 2) {
            int p, q;
            bj_pair(BJ_W, rr, tid, p, q);
            const double al = M[p * BJ_MLD + p], be = M[q * BJ_MLD + q], ga = M[p * BJ_MLD + q];
            double c = 1.0, s = 0.0;
            // the per-round chain is latency-bound: MUFU approximations + one Newton step each
            // instead of IEEE div / sqrt (relative error ~1e-15, far below the sweep tolerance)
            if (al * be > 0.0 && ga * ga > 1e-30 * (al * be)) {
                const double zeta = (be - al) * 0.5 * bj_rcp(ga);
                const double z2 = fma(zeta, zeta, 1.0);
                const double sq = z2 * bj_rsqrt(z2);   // sqrt(1 + zeta^2)
                const double t = copysign(bj_rcp(fabs(zeta) + sq), zeta);
                c = bj_rsqrt(fma(t, t, 1.0));
                s = c * t;
            }
            // w_p' = c w_p - s w_q,  w_q' = s w_p + c w_q
            s_a[p] = c;
            s_b[p] = -s;
            s_o[p] = q;
            s_a[q] = c;
            s_b[q] = s;
            s_o[q] = p;
        }
        __syncthreads();
        // M <- J^T M J on 2 x 2 blocks {i, o_i} x {j, o_j} (each block updated by one thread, in place)
        for (int e = tid; e < (BJ_W / 2) * (BJ_W / 2); e += BJ_THREADS) {
            const int ti = e / (BJ_W / 2), tj = e % (BJ_W / 2);
            int i, oi, j, oj;
            bj_pair(BJ_W, rr, ti, i, oi);
            bj_pair(BJ_W, rr, tj, j, oj);
            const double m00 = M[i * BJ_MLD + j], m01 = M[i * BJ_MLD + oj];
            const double m10 = M[oi * BJ_MLD + j], m11 = M[oi * BJ_MLD + oj];
            const double ai = s_a[i], bi = s_b[i], aoi = s_a[oi], boi = s_b[oi];
            const double aj = s_a[j], bj = s_b[j], aoj = s_a[oj], boj = s_b[oj];
            // column rotation then row rotation: (x' = a_x x + b_x x_partner)
            const double c00 = aj * m00 + bj * m01, c01 = aoj * m01 + boj * m00;
            const double c10 = aj * m10 + bj * m11, c11 = aoj * m11 + boj * m10;
            M[i * BJ_MLD + j] = ai * c00 + bi * c10;
            M[i * BJ_MLD + oj] = ai * c01 + bi * c11;
            M[oi * BJ_MLD + j] = aoi * c10 + boi * c00;
            M[oi * BJ_MLD + oj] = aoi * c11 + boi * c01;
        }
        // U <- U J (rows x pairs, in place)
        for (int e = tid; e < BJ_W * (BJ_W / 2); e += BJ_THREADS) {
            const int r = e / (BJ_W / 2), t = e % (BJ_W / 2);
            int p, q;
            bj_pair(BJ_W, rr, t, p, q);
            const double up = U[r * BJ_ULD + p], uq = U[r * BJ_ULD + q];
            U[r * BJ_ULD + p] = s_a[p] * up + s_b[p] * uq;
            U[r * BJ_ULD + q] = s_a[q] * uq + s_b[q] * up;
        }
        __syncthreads();
    }
    // ---- 5. W_IJ <- W_IJ U on DMMA: warp w owns rows 8 w .. 8 w + 7 (all 64 output columns)
    for (int rb = warp; 8 * rb < rows4; rb += BJ_NW) {
        const int g = lane >> 2, c = lane & 3;
        double acc[BJ_NB8][2];
#pragma unroll
        for (int ct = 0; ct < BJ_NB8; ++ct) acc[ct][0] = acc[ct][1] = 0.0;
#pragma unroll 4
        for (int k0 = 0; k0 < BJ_W; k0 += 4) {
            const double av = Ws[(k0 + c) * a.lds + 8 * rb + g];   // A(g, c) = W(row 8 rb + g, col k0 + c)
#pragma unroll
            for (int ct = 0; ct < BJ_NB8; ++ct) bj_dmma(acc[ct], av, U[(k0 + c) * BJ_ULD + 8 * ct + g]);
        }
        __syncwarp();
#pragma unroll
        for (int ct = 0; ct < BJ_NB8; ++ct) {
            Ws[(8 * ct + 2 * c) * a.lds + 8 * rb + g] = acc[ct][0];
            Ws[(8 * ct + 2 * c + 1) * a.lds + 8 * rb + g] = acc[ct][1];
        }
    }
    __syncthreads();
    // ---- 6. store
    for (int e = tid; e < BJ_W * rows; e += BJ_THREADS) {
        const int lc = e / rows, i = e % rows;
        const int gc = lc < BJ_B ? bI * BJ_B + lc : bJ * BJ_B + (lc - BJ_B);
        a.W[(int64_t)gc * a.l + r0 + i] = Ws[lc * a.lds + i];
    }
    cl.sync();   // no CTA leaves while a cluster peer may still read its shared memory
}

bool svd_bj_fits(int l) {
    if (getenv("RGSQR_JACOBI_SCALAR") != nullptr) return false;
    const int min_l = getenv("RGSQR_JACOBI_BLOCK_MIN") ? atoi(getenv("RGSQR_JACOBI_BLOCK_MIN")) : 545;
    return l >= min_l && l >= 2 && l <= 8 * BJ_MAX_ROWS;
}

int svd_bj_cols(int l) { return ((l + BJ_W - 1) / BJ_W) * BJ_W; }

// W: l x svd_bj_cols(l) fp64 (ld l), initialised (padding columns zero).  maxoff: >= max_sweeps
// uint64 of device memory.  Runs until the max off-diagonal ratio of a sweep is below tol (checked
// on the host every sweep) or max_sweeps; *sweeps_out = sweeps run.
cudaError_t launch_svd_bj(double* W, int l, int max_sweeps, double tol, unsigned long long* maxoff, int* sweeps_out,
                          cudaStream_t st) {
    const int nblk = svd_bj_cols(l) / BJ_B;
    const int P = nblk / 2;
    int C = 1;
    while (C < 8 && (P * C * 2 <= 148 || (l + C - 1) / C > BJ_MAX_ROWS)) C *= 2;   // ~128-148 CTAs
    const int rpc = (l + C - 1) / C;
    if (rpc > BJ_MAX_ROWS) return cudaErrorInvalidValue;
    const int rows8 = (rpc + 7) & ~7;
    const int lds = ((rows8 - 4 + 15) & ~15) + 4;   // == 4 mod 16 doubles, >= rows8
    const size_t smem = ((size_t)BJ_W * lds + 2 * BJ_NE + BJ_W * BJ_MLD + BJ_W * BJ_ULD + BJ_NT * 64) * 8;
    cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(svd_bj_round_kernel), smem);
    if (e != cudaSuccess) return e;
    e = cudaMemsetAsync(maxoff, 0, sizeof(unsigned long long) * max_sweeps, st);
    if (e != cudaSuccess) return e;
    BjArgs a{};
    a.W = W;
    a.l = l;
    a.nblk = nblk;
    a.C = C;
    a.rpc = rpc;
    a.lds = lds;
    a.tol = tol;
    a.maxoff = maxoff;
    cudaLaunchConfig_t cfg{};
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = C;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.gridDim = dim3(P * C);
    cfg.blockDim = dim3(BJ_THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int sweep = 0;
    for (; sweep < max_sweeps; ++sweep) {
        a.sweep = sweep;
        for (int r = 0; r < nblk - 1; ++r) {
            a.round = r;
            ++g_launches;
            e = cudaLaunchKernelEx(&cfg, svd_bj_round_kernel, a);
            if (e != cudaSuccess) return e;
        }
        // convergence: the max off-diagonal ratio seen at the start of this sweep's pair updates
        unsigned long long bits = 0;
        e = cudaMemcpyAsync(&bits, maxoff + sweep, sizeof(bits), cudaMemcpyDeviceToHost, st);
        if (e != cudaSuccess) return e;
        e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) return e;
        double mx;
        memcpy(&mx, &bits, sizeof(mx));
        if (getenv("RGSQR_JACOBI_TRACE")) fprintf(stderr, "[rgsqr svd] sweep %d: max off-diagonal cosine %.3e\n", sweep, mx);
        if (mx < tol) {
            ++sweep;
            break;
        }
    }
    if (sweeps_out) *sweeps_out = sweep;
    return cudaSuccess;
}

}  // namespace rg
