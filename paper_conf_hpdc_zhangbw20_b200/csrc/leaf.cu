// leaf.cu -- the last level of Algorithm 1 in one kernel: for a block
// of nc <= 64 columns split as h = min(32, nc), w = nc - h,
//
//   [Q1, R11] = panel(P1)                      (Alg 1 line 6; CholQR, fp64 Gram)
//   R12       = Q1^T P2                        (line 8, 16-bit operands, fp32 accumulation)
//   P2       <- P2 - Q1 R12                    (line 9, same precision)
//   [Q2, R22] = panel(P2)                      (line 10)
//
// with the block's rows resident in shared memory: every CTA of a cooperative grid (one per SM)
// owns a contiguous run of rows, loads them once (cp.async), and writes Q (fp32 + 16-bit shadow)
// once.  The three cross-row reductions (the two Gram matrices and R12) are deterministic grid
// all-reductions: each CTA writes its partial, a grid barrier, CTA b sums entry slice b over all
// partials in CTA order (one warp per entry, fixed shuffle tree), a second barrier, and every CTA
// reads the reduced result.
//
// Why a new kernel ("Leaf"): on B200 the 65536 x 32 panel is a few us of
// HBM traffic, so the leaf level is latency-bound.  Measured with per-op events at config 2, the
// previous structure (K1 GEMM + split-K reduce + a fused CholQR2 panel with the leaf K2 folded
// in) cost ~118 us per 64 columns.  The pieces here are built for latency:
//   * Gram on the fp64 tensor cores (DMMA m8n8k4) straight from the fp32 rows in smem (one
//     fragment per 8-column block serves as both A and B), no staging copy;
//   * K1 / K2 of the leaf level on mma.sync m16n8k16 (fp16 or bf16 in, fp32 accumulate -- the
//     precision of the tensor-core GEMMs of the upper levels);
//   * the 32 x 32 Cholesky in one warp, fp64, column j in lane j's registers (32 dependent
//     pivots, no block barriers), then R^{-1} by column-parallel back substitution;
//   * P <- P R^{-1} exploiting the triangle (warp-uniform column groups).
// Panel numerics are those of panel_cholqr.cu: one CholQR pass when kappa_F(R1) <= 2 nc, else
// CholQR2; a failed pivot switches to shifted CholQR3 (shift 11 (m nc + nc (nc + 1)) u ||P||_F^2);
// a pivot that still fails is a numerical breakdown reported through status (col0 + j).
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>

#include <cstdlib>

#include "kernels.h"
#include "ptx.cuh"

namespace rg {

constexpr int LF_THREADS = 512;
constexpr int LF_NW = LF_THREADS / 32;
constexpr int LF_MAXI = 9;                   // row groups of 64 per thread in the apply (<= 576 rows)
constexpr int LF_GLD = 34;                   // fp64 32 x 32 matrices in smem: row stride (16-byte rows)
constexpr int LF_R12LD = 40;                 // 16-bit R12 image [n][k] row stride (halves)
constexpr int LF_SCRATCH = 5120;             // doubles of warp-partial scratch (40 KB)
constexpr int LF_PART = 1024;                // doubles per CTA partial in the workspace
constexpr int LF_MAX_GRID = 160;

struct LeafArgs {
    float* Q;            // block columns: in = P (after the upper levels' updates), out = Q; fp32, ldq
    int64_t ldq;
    uint16_t* Qh;        // 16-bit shadow of Q (hi), ldh; may be null
    uint16_t* Ql;        // lo part (split mode) or null
    int64_t ldh;
    int64_t m;           // rows (global)
    int nc;              // block columns, 1..64
    float* R;            // nc x nc diagonal block of R, ldr (upper written, lower zeroed)
    int64_t ldr;
    double* part;        // [LF_MAX_GRID][LF_PART] CTA partials
    double* red;         // [LF_PART] reduced result
    unsigned* bar;       // grid barrier word (generation bit flips every barrier)
    int* status;         // atomicMin(status, col0 + j) on a numerical breakdown
    int col0;
    int bf16;
    int rows_per;        // rows per CTA (multiple of 8)
    int ldt;             // smem tile leading dimension (floats), == 4 mod 32
    int vec;             // 16-byte global accesses allowed
};

#ifdef LF_TRACE
__device__ unsigned long long lf_trace[32];
#define LF_MARK(i)                                                                     \
    do {                                                                               \
        if (blockIdx.x == 0 && threadIdx.x == 0) {                                     \
            unsigned long long t_;                                                     \
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                     \
            lf_trace[i] = t_;                                                          \
        }                                                                              \
    } while (0)
#else
#define LF_MARK(i) \
    do {           \
    } while (0)
#endif

// ------------------------------------------------------------------ small helpers
__device__ __forceinline__ unsigned lf_ld_acquire(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Grid-wide barrier for a cooperative launch (all CTAs co-resident).  The word is never reset:
// CTA 0 adds 2^31 - (grid - 1) and every other CTA 1, so each barrier adds exactly 2^31 and its
// completion is the flip of the top bit relative to the value this CTA saw on arrival.
__device__ __forceinline__ void lf_grid_sync(unsigned* bar) {
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned nb = (blockIdx.x == 0) ? (0x80000000u - (gridDim.x - 1)) : 1u;
        __threadfence();
        const unsigned old = atomicAdd(bar, nb);
        while (((lf_ld_acquire(bar) ^ old) & 0x80000000u) == 0) {
        }
        __threadfence();
    }
    __syncthreads();
}

__device__ __forceinline__ void lf_cp16(float* sdst, const float* gsrc, int src_bytes) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(sdst)), "l"(gsrc), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void lf_cp4(float* sdst, const float* gsrc, int src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(smem_u32(sdst)), "l"(gsrc), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void lf_cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void lf_cp_wait() {
    asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

__device__ __forceinline__ uint32_t lf_pack2(float lo, float hi, int bf16) {
    if (bf16) {
        __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
        return *reinterpret_cast<uint32_t*>(&v);
    }
    __half2 v = __floats2half2_rn(lo, hi);
    return *reinterpret_cast<uint32_t*>(&v);
}
__device__ __forceinline__ uint16_t lf_to16(float x, int bf16) {
    if (bf16) {
        __nv_bfloat16 b = __float2bfloat16_rn(x);
        return *reinterpret_cast<uint16_t*>(&b);
    }
    __half h = __float2half_rn(x);
    return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float lf_from16(uint16_t u, int bf16) {
    if (bf16) return __bfloat162float(*reinterpret_cast<__nv_bfloat16*>(&u));
    return __half2float(*reinterpret_cast<__half*>(&u));
}

// D += A B on the 16-bit tensor cores: m16n8k16, fp32 accumulate.
__device__ __forceinline__ void lf_mma16816(float (&d)[4], const uint32_t (&a)[4], const uint32_t (&b)[2], int bf16) {
    if (bf16)
        asm volatile(
            "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
            "{%0,%1,%2,%3};"
            : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
            : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
    else
        asm volatile(
            "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
            "{%0,%1,%2,%3};"
            : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
            : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
}

// ------------------------------------------------------------------ shared memory
struct LfSmem {
    float* tile;      // 64 columns x ldt rows (fp32, column-major)
    double* scr;      // LF_SCRATCH doubles: warp partials
    double* G;        // 32 x LF_GLD: reduced Gram (full symmetric), then Cholesky scratch
    double* Rs;       // 32 x LF_GLD: R of the current pass, row-major R(i, j) = Rs[i * LD + j]
    double* Racc;     // 32 x LF_GLD: accumulated R of the panel (R_p ... R_1)
    double* Rt;       // 32 x LF_GLD: R of the current pass, column-major R(i, j) = Rt[j * LD + i]
    double* U;        // 32 x LF_GLD: row k of the Schur complement at elimination step k
    float* Rt32;      // 32 x 36: fp32 copy of R, column-major (inverse input)
    float* rdiag32;   // 32
    int* pivok;       // 32: pivot k accepted
    double* red;      // 1024: reduced values of the current all-reduction
    double* rdiag;    // 32: 1 / R(k, k)
    float* Ri;        // 32 x 32 fp32 R^{-1}, row-major
    uint16_t* R12h;   // 32 x LF_R12LD: -R12 as the K2 B operand, [n][k]
    static constexpr size_t fixed_bytes() {
        return (size_t)LF_SCRATCH * 8 + 5 * 32 * LF_GLD * 8 + 1024 * 8 + 32 * 8 + 32 * 4 + 32 * 36 * 4 + 32 * 4 + 32 * 32 * 4 + 32 * LF_R12LD * 2 + 256;
    }
    __device__ LfSmem(uint8_t* base, int ldt) {
        tile = reinterpret_cast<float*>(base);
        uint8_t* p = base + (size_t)64 * ldt * 4;
        scr = reinterpret_cast<double*>(p);
        p += (size_t)LF_SCRATCH * 8;
        G = reinterpret_cast<double*>(p);
        p += 32 * LF_GLD * 8;
        Rs = reinterpret_cast<double*>(p);
        p += 32 * LF_GLD * 8;
        Racc = reinterpret_cast<double*>(p);
        p += 32 * LF_GLD * 8;
        Rt = reinterpret_cast<double*>(p);
        p += 32 * LF_GLD * 8;
        U = reinterpret_cast<double*>(p);
        p += 32 * LF_GLD * 8;
        Rt32 = reinterpret_cast<float*>(p);
        p += 32 * 36 * 4;
        rdiag32 = reinterpret_cast<float*>(p);
        p += 32 * 4;
        red = reinterpret_cast<double*>(p);
        p += 1024 * 8;
        rdiag = reinterpret_cast<double*>(p);
        p += 32 * 8;
        pivok = reinterpret_cast<int*>(p);
        p += 32 * 4;
        Ri = reinterpret_cast<float*>(p);
        p += 32 * 32 * 4;
        R12h = reinterpret_cast<uint16_t*>(p);
    }
};

// ------------------------------------------------------------------ grid all-reduction
// Sum of the CTA partials part[b][0, ne) (already written by this CTA) into s.red on every CTA.
// Deterministic: entry e is summed by one warp of CTA e / slice, lanes over CTAs lane, lane + 32,
// ... in order, then a fixed xor-shuffle tree.
__device__ void lf_allreduce(const LeafArgs& a, const LfSmem& s, int ne) {
    lf_grid_sync(a.bar);
    const int grid = gridDim.x;
    const int slice = (ne + grid - 1) / grid;   // entries per CTA (<= LF_NW for ne <= 1024, grid >= 64)
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int q = warp; q < slice; q += LF_NW) {
        const int e = blockIdx.x * slice + q;
        if (e < ne) {
            double v = 0.0;
            for (int b = lane; b < grid; b += 32) v += __ldcg(a.part + (int64_t)b * LF_PART + e);
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
            if (lane == 0) __stcg(a.red + e, v);
        }
    }
    lf_grid_sync(a.bar);
    for (int e = threadIdx.x; e < ne; e += LF_THREADS) s.red[e] = __ldcg(a.red + e);
    __syncthreads();
}

// ------------------------------------------------------------------ Gram (fp64 tensor cores)
// Partial G = P^T P of the CTA's rows [0, rp) of tile columns [c0, c0 + 32), written packed
// (upper triangle, [j (j + 1) / 2 + i]) into this CTA's workspace partial.
__device__ void lf_gram(const LeafArgs& a, const LfSmem& s, int c0, int rp) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, c = lane & 3;
    double acc[10][2];
#pragma unroll
    for (int t = 0; t < 10; ++t) acc[t][0] = acc[t][1] = 0.0;
    const float* col = s.tile + (int64_t)(c0 + g) * a.ldt + c;
    for (int k0 = 4 * warp; k0 < rp; k0 += 4 * LF_NW) {
        double f[4];
#pragma unroll
        for (int b = 0; b < 4; ++b) f[b] = (double)col[8 * b * a.ldt + k0];
        int t = 0;
#pragma unroll
        for (int bi = 0; bi < 4; ++bi)
#pragma unroll
            for (int bj = bi; bj < 4; ++bj, ++t)
                asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                             : "+d"(acc[t][0]), "+d"(acc[t][1])
                             : "d"(f[bi]), "d"(f[bj]));
    }
    // warp partials summed in warp order: two rounds of 8 warps through the scratch
    constexpr int NENT = 640;   // 10 blocks x 64
    double run[2] = {0.0, 0.0};
    for (int w0 = 0; w0 < LF_NW; w0 += 8) {
        __syncthreads();
        if (warp >= w0 && warp < w0 + 8) {
            double* dst = s.scr + (warp - w0) * NENT + lane;
#pragma unroll
            for (int t = 0; t < 10; ++t) {
                dst[(2 * t) * 32] = acc[t][0];
                dst[(2 * t + 1) * 32] = acc[t][1];
            }
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            const int e = threadIdx.x + LF_THREADS * q;
            if (e < NENT)
#pragma unroll
                for (int k = 0; k < 8; ++k) run[q] += s.scr[k * NENT + e];
        }
    }
    // entry e = (2 t + u) * 32 + ln of block t = (bi, bj): G(8 bi + ln / 4, 8 bj + 2 (ln % 4) + u)
    double* out = a.part + (int64_t)blockIdx.x * LF_PART;
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int e = threadIdx.x + LF_THREADS * q;
        if (e < NENT) {
            const int t = e >> 6, u = (e >> 5) & 1, ln = e & 31;
            int bi = 0, tt = t;
            while (tt >= 4 - bi) {
                tt -= 4 - bi;
                ++bi;
            }
            const int bj = bi + tt;
            const int i = 8 * bi + (ln >> 2), j = 8 * bj + 2 * (ln & 3) + u;
            if (i <= j) __stcg(out + j * (j + 1) / 2 + i, run[q]);
        }
    }
}

// ------------------------------------------------------------------ Cholesky + inverse (warp 0)
// fp64 1/sqrt: hardware approximation + one Newton step (relative error ~2^-44, far below what
// the fp32 outputs can resolve; the pivot test is done on d itself).
__device__ __forceinline__ double lf_rsqrt(double d) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(d));
    const double e = fma(-d * y, y, 1.0);
    return fma(0.5 * y, e, y);
}

// s.G holds the full symmetric 32 x 32 Gram (identity beyond nc).  Lane j keeps column j of the
// Schur complement S in registers.  Step k: every lane publishes S(k, j) (row k, through s.U),
// then every lane reads the whole row back with 16-byte broadcasts and computes the pivot itself
// (rs = 1 / sqrt(S(k, k)): one shared-memory round trip per step and no branch on the pivot
// lane), forms R(k, j) = S(k, j) rs and updates S(i, j) -= S(k, i) S(k, j) / S(k, k), the next
// pivot's entry first.  Measured on B200 (one warp): DFMA issue 2.6 cycles, DFMA latency 8.7,
// STS + syncwarp + LDS 44, rsqrt (approx + Newton) 48; the whole factorization ~7.5K cycles.
// (Shuffles inside the warp-0 branch compile to WARPSYNC / ENDCOLLECTIVE sequences, ~2x slower;
// a fraction-free variant without the division on the chain triples the fp64 work per element
// and was slower, 9.4K cycles.)  Writes s.Rs (row-major R), s.Rt and s.Rt32 (column-major R, fp64
// / fp32), s.rdiag / s.rdiag32 (1 / R(k, k)).  Returns the first failed pivot (32 if none): a
// pivot fails unless it is finite and > 1e-15 G(k, k).
__device__ int lf_chol_warp(const LfSmem& s) {
    const int lane = threadIdx.x & 31;
    double g[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) g[i] = s.G[i * LF_GLD + lane];
    int bad = 32;
#pragma unroll
    for (int k = 0; k < 32; ++k) {
        double* urow = s.U + k * LF_GLD;
        urow[lane] = g[k];
        __syncwarp();
        const double d = urow[k];
        const bool good = (d > s.G[k * LF_GLD + k] * 1e-15) && isfinite(d);
        bad = (!good && bad == 32) ? k : bad;
        const double rs = good ? lf_rsqrt(d) : 1.0;
        const double r = (lane >= k) ? g[k] * rs : 0.0;   // R(k, lane); lane k: sqrt(d)
        const double t = r * rs;                           // S(k, lane) / S(k, k)
        if (k + 1 < 32) g[k + 1] = fma(-urow[k + 1], t, g[k + 1]);
        if ((k & 1) == 0) {   // k + 2 even: pairs from k + 2
#pragma unroll
            for (int i = k + 2; i < 32; i += 2) {
                const double2 v = *reinterpret_cast<const double2*>(urow + i);
                g[i] = fma(-v.x, t, g[i]);
                g[i + 1] = fma(-v.y, t, g[i + 1]);
            }
        } else {              // k + 2 odd: one scalar, then pairs
            if (k + 2 < 32) g[k + 2] = fma(-urow[k + 2], t, g[k + 2]);
#pragma unroll
            for (int i = k + 3; i < 32; i += 2) {
                const double2 v = *reinterpret_cast<const double2*>(urow + i);
                g[i] = fma(-v.x, t, g[i]);
                g[i + 1] = fma(-v.y, t, g[i + 1]);
            }
        }
        s.Rs[k * LF_GLD + lane] = r;
        s.Rt[lane * LF_GLD + k] = r;
        s.Rt32[lane * 36 + k] = (float)r;
        if (lane == 0) {
            s.rdiag[k] = rs;
            s.rdiag32[k] = (float)rs;
        }
    }
    __syncwarp();
    return bad;
}

// X = R^{-1} (upper) in fp32 (it only feeds the fp32 product P R^{-1} and the kappa test), lane j
// computes column j by back substitution: right-looking, each step one multiply and independent
// FMAs, column k of R read from s.Rt32 with 16-byte broadcasts.  Writes s.Ri (row-major) and
// returns |R|_F^2 |R^{-1}|_F^2 over the nc x nc panel.
__device__ double lf_inverse_warp(const LfSmem& s, int nc) {
    const int lane = threadIdx.x & 31;
    float b[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) b[i] = (i == lane) ? 1.f : 0.f;
#pragma unroll
    for (int k = 31; k >= 0; --k) {
        b[k] *= s.rdiag32[k];
        const float* col = s.Rt32 + k * 36;
#pragma unroll
        for (int i = 0; i + 3 < k; i += 4) {
            const float4 v = *reinterpret_cast<const float4*>(col + i);
            b[i] = fmaf(-v.x, b[k], b[i]);
            b[i + 1] = fmaf(-v.y, b[k], b[i + 1]);
            b[i + 2] = fmaf(-v.z, b[k], b[i + 2]);
            b[i + 3] = fmaf(-v.w, b[k], b[i + 3]);
        }
#pragma unroll
        for (int i = k & ~3; i < k; ++i) b[i] = fmaf(-col[i], b[k], b[i]);
    }
    double xn = 0.0, rn = 0.0;
#pragma unroll
    for (int i = 0; i < 32; ++i) {
        s.Ri[i * 32 + lane] = b[i];
        const double r = s.Rs[i * LF_GLD + lane];
        if (i < nc && lane < nc) {   // the identity padding beyond nc is not part of the panel
            xn = fma((double)b[i], (double)b[i], xn);
            rn = fma(r, r, rn);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        xn += __shfl_xor_sync(0xffffffffu, xn, o);
        rn += __shfl_xor_sync(0xffffffffu, rn, o);
    }
    __syncwarp();
    return xn * rn;
}

// Racc <- Rs * Racc (first pass: Racc = Rs); lane j owns column j.
__device__ void lf_racc_warp(const LfSmem& s, bool first) {
    const int lane = threadIdx.x & 31;
    double v[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) {
        if (first) {
            v[i] = s.Rs[i * LF_GLD + lane];
        } else {
            double acc = 0.0;
#pragma unroll 1
            for (int k = i; k < 32; ++k) acc = fma(s.Rs[i * LF_GLD + k], s.Racc[k * LF_GLD + lane], acc);
            v[i] = acc;
        }
    }
    __syncwarp();
#pragma unroll
    for (int i = 0; i < 32; ++i) s.Racc[i * LF_GLD + lane] = v[i];
    __syncwarp();
}

// tile columns [c0, c0 + 32), rows [0, rp) <- tile * R^{-1} (fp32).  Warp w takes the column
// group cg = w % 8 (4 columns) and the rows (w / 8) * 32 + lane + 64 i (i < NI); R^{-1} is upper,
// so the k loop stops at the group's last column (warp-uniform).
template <int NI>
__device__ void lf_apply(const LeafArgs& a, const LfSmem& s, int c0, int rp) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int cg = warp & 7, half = warp >> 3;
    const int ld = a.ldt;
    const int r0 = half * 32 + lane;
    float o[NI][4];
#pragma unroll
    for (int i = 0; i < NI; ++i)
#pragma unroll
        for (int c = 0; c < 4; ++c) o[i][c] = 0.f;
    const float* base = s.tile + c0 * ld + r0;
    const int kend = 4 * cg + 4;
    int off = 0;
#pragma unroll 4
    for (int k = 0; k < kend; ++k, off += ld) {
        const float4 rv = *reinterpret_cast<const float4*>(s.Ri + k * 32 + 4 * cg);
#pragma unroll
        for (int i = 0; i < NI; ++i) {
            const float x = base[off + 64 * i];   // rows >= rp hold zeros (loaded as zero-fill)
            o[i][0] = fmaf(x, rv.x, o[i][0]);
            o[i][1] = fmaf(x, rv.y, o[i][1]);
            o[i][2] = fmaf(x, rv.z, o[i][2]);
            o[i][3] = fmaf(x, rv.w, o[i][3]);
        }
    }
    __syncthreads();
    float* ob = s.tile + (c0 + 4 * cg) * ld + r0;
#pragma unroll
    for (int i = 0; i < NI; ++i)
        if (r0 + 64 * i < rp)
#pragma unroll
            for (int c = 0; c < 4; ++c) ob[c * ld + 64 * i] = o[i][c];
    __syncthreads();
}

// CholQR of the panel in tile columns [c0, c0 + 32) (nc valid columns, the rest zero) with the
// single-pass test, CholQR2 and the shifted-CholQR3 fallback.  Leaves Q in the tile and R in
// s.Racc (fp64, row-major).  Returns the first failed pivot column (or -1).
template <int NI>
__device__ int lf_panel(const LeafArgs& a, const LfSmem& s, int c0, int nc, int rp, int tb) {
    __shared__ int s_flag[2];
    bool shifted = false;
    int bad = -1;
    for (int pass = 0; pass < 3; ++pass) {
        lf_gram(a, s, c0, rp);
        if (pass == 0) LF_MARK(tb + 0);
        lf_allreduce(a, s, 528);
        if (pass == 0) LF_MARK(tb + 1);
        // full symmetric Gram, identity beyond nc
        for (int e = threadIdx.x; e < 1024; e += LF_THREADS) {
            const int i = e >> 5, j = e & 31;
            const int lo = min(i, j), hi = max(i, j);
            s.G[i * LF_GLD + j] = (i < nc && j < nc) ? s.red[hi * (hi + 1) / 2 + lo] : (i == j ? 1.0 : 0.0);
        }
        __syncthreads();
        if (threadIdx.x < 32) {
            int fb = lf_chol_warp(s);
            if (fb < 32 && pass == 0) {
                // shifted CholQR: G + sh I, sh = 11 (m nc + nc (nc + 1)) u ||P||_F^2
                double tr = 0.0;
                for (int e = threadIdx.x; e < nc; e += 32) {
                    const int hi = e;
                    tr += s.red[hi * (hi + 1) / 2 + hi];
                }
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) tr += __shfl_xor_sync(0xffffffffu, tr, o);
                const double sh = 11.0 * ((double)a.m * nc + (double)nc * (nc + 1)) * 0x1p-53 * tr;
                const int lane = threadIdx.x;
                if (lane < nc) s.G[lane * LF_GLD + lane] += sh;
                __syncwarp();
                fb = lf_chol_warp(s);
                if (threadIdx.x == 0) s_flag[1] = 1;
            } else if (threadIdx.x == 0) {
                s_flag[1] = 0;
            }
            if (fb < 32) {
                if (threadIdx.x == 0) s_flag[0] = -(fb + 1);
            } else {
                const double kk = lf_inverse_warp(s, nc);
                lf_racc_warp(s, pass == 0);
                if (threadIdx.x == 0) s_flag[0] = (kk <= 4.0 * nc * nc) ? 1 : 0;   // kappa_F <= 2 nc
            }
        }
        __syncthreads();
        if (pass == 0) LF_MARK(tb + 2);
        if (s_flag[1]) shifted = true;
        const int f = s_flag[0];
        if (f < 0) {
            bad = -f - 1;
            break;
        }
        bool stop;
        if (pass == 0)
            stop = !shifted && f == 1;
        else
            stop = (pass == 1 && !shifted) || pass == 2;
        lf_apply<NI>(a, s, c0, rp);
        if (pass == 0) LF_MARK(tb + 3);
        if (stop) break;
    }
    return bad;
}

// ------------------------------------------------------------------ K1 / K2 of the leaf level
// Partial R12 = Q1^T P2 (tile columns [0, 32) and [32, 64)) on the 16-bit tensor cores.
__device__ void lf_k1(const LeafArgs& a, const LfSmem& s, int rp16) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, c = lane & 3;
    float acc[2][4][4];
#pragma unroll
    for (int mt = 0; mt < 2; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt)
#pragma unroll
            for (int u = 0; u < 4; ++u) acc[mt][nt][u] = 0.f;
    const int ld = a.ldt;
    for (int k0 = 16 * warp; k0 < rp16; k0 += 16 * LF_NW) {
        uint32_t af[2][4], bfr[4][2];
#pragma unroll
        for (int mt = 0; mt < 2; ++mt) {
            const float* q = s.tile + (int64_t)(16 * mt + g) * ld + k0 + 2 * c;
            const float2 x0 = *reinterpret_cast<const float2*>(q);
            const float2 x1 = *reinterpret_cast<const float2*>(q + 8 * ld);
            const float2 x2 = *reinterpret_cast<const float2*>(q + 8);
            const float2 x3 = *reinterpret_cast<const float2*>(q + 8 * ld + 8);
            af[mt][0] = lf_pack2(x0.x, x0.y, a.bf16);
            af[mt][1] = lf_pack2(x1.x, x1.y, a.bf16);
            af[mt][2] = lf_pack2(x2.x, x2.y, a.bf16);
            af[mt][3] = lf_pack2(x3.x, x3.y, a.bf16);
        }
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
            const float* p = s.tile + (int64_t)(32 + 8 * nt + g) * ld + k0 + 2 * c;
            const float2 y0 = *reinterpret_cast<const float2*>(p);
            const float2 y1 = *reinterpret_cast<const float2*>(p + 8);
            bfr[nt][0] = lf_pack2(y0.x, y0.y, a.bf16);
            bfr[nt][1] = lf_pack2(y1.x, y1.y, a.bf16);
        }
#pragma unroll
        for (int mt = 0; mt < 2; ++mt)
#pragma unroll
            for (int nt = 0; nt < 4; ++nt) lf_mma16816(acc[mt][nt], af[mt], bfr[nt], a.bf16);
    }
    // warp partials in warp order (two rounds of 8) -> CTA partial (as doubles)
    float* scr = reinterpret_cast<float*>(s.scr);
    double run[2] = {0.0, 0.0};
    for (int w0 = 0; w0 < LF_NW; w0 += 8) {
        __syncthreads();
        if (warp >= w0 && warp < w0 + 8) {
            float* dst = scr + (warp - w0) * 1024 + lane;
#pragma unroll
            for (int mt = 0; mt < 2; ++mt)
#pragma unroll
                for (int nt = 0; nt < 4; ++nt)
#pragma unroll
                    for (int u = 0; u < 4; ++u) dst[((mt * 4 + nt) * 4 + u) * 32] = acc[mt][nt][u];
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            const int e = threadIdx.x + LF_THREADS * q;
#pragma unroll
            for (int k = 0; k < 8; ++k) run[q] += (double)scr[k * 1024 + e];
        }
    }
    // entry e = ((mt * 4 + nt) * 4 + u) * 32 + ln: R12(16 mt + ln / 4 + 8 (u / 2), 8 nt + 2 (ln % 4) + u % 2)
    double* out = a.part + (int64_t)blockIdx.x * LF_PART;
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int e = threadIdx.x + LF_THREADS * q;
        const int ln = e & 31, u = (e >> 5) & 3, nt = (e >> 7) & 3, mt = e >> 9;
        const int i = 16 * mt + (ln >> 2) + 8 * (u >> 1), j = 8 * nt + 2 * (ln & 3) + (u & 1);
        __stcg(out + i * 32 + j, run[q]);
    }
}

// P2 <- P2 - Q1 R12 (tile columns [32, 64) -= [0, 32) * R12) with 16-bit operands; s.R12h holds
// -R12 as [n][k].
__device__ void lf_k2(const LeafArgs& a, const LfSmem& s, int rp16) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, c = lane & 3;
    const int ld = a.ldt;
    uint32_t bfr[2][4][2];
#pragma unroll
    for (int ks = 0; ks < 2; ++ks)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
            const uint16_t* bp = s.R12h + (8 * nt + g) * LF_R12LD + 16 * ks + 2 * c;
            bfr[ks][nt][0] = *reinterpret_cast<const uint32_t*>(bp);
            bfr[ks][nt][1] = *reinterpret_cast<const uint32_t*>(bp + 8);
        }
    for (int r0 = 16 * warp; r0 < rp16; r0 += 16 * LF_NW) {
        float d[4][4];
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
            const float* cp = s.tile + (int64_t)(32 + 8 * nt + 2 * c) * ld + r0 + g;
            d[nt][0] = cp[0];
            d[nt][1] = cp[ld];
            d[nt][2] = cp[8];
            d[nt][3] = cp[ld + 8];
        }
#pragma unroll
        for (int ks = 0; ks < 2; ++ks) {
            const float* q = s.tile + (int64_t)(16 * ks + 2 * c) * ld + r0 + g;
            uint32_t af[4];
            af[0] = lf_pack2(q[0], q[ld], a.bf16);
            af[1] = lf_pack2(q[8], q[ld + 8], a.bf16);
            af[2] = lf_pack2(q[8 * ld], q[9 * ld], a.bf16);
            af[3] = lf_pack2(q[8 * ld + 8], q[9 * ld + 8], a.bf16);
#pragma unroll
            for (int nt = 0; nt < 4; ++nt) lf_mma16816(d[nt], af, bfr[ks][nt], a.bf16);
        }
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
            float* cp = s.tile + (int64_t)(32 + 8 * nt + 2 * c) * ld + r0 + g;
            cp[0] = d[nt][0];
            cp[ld] = d[nt][1];
            cp[8] = d[nt][2];
            cp[ld + 8] = d[nt][3];
        }
    }
    __syncthreads();
}

// ------------------------------------------------------------------ load / store
__device__ void lf_load_cols(const LeafArgs& a, const LfSmem& s, int64_t r0, int rows, int rp16, int cbeg, int cend) {
    const int nq = rp16 >> 2;   // 4-row chunks per column
    const int total = (cend - cbeg) * nq;
    for (int e = threadIdx.x; e < total; e += LF_THREADS) {
        const int cc = cbeg + e / nq, q = e % nq;
        float* dst = s.tile + (int64_t)cc * a.ldt + 4 * q;
        const float* src = a.Q + r0 + (int64_t)cc * a.ldq;
        const int avail = (cc < a.nc) ? max(0, min(4, rows - 4 * q)) : 0;
        if (a.vec) {
            lf_cp16(dst, avail > 0 ? src + 4 * q : src, avail * 4);
        } else {
#pragma unroll
            for (int u = 0; u < 4; ++u) lf_cp4(dst + u, (u < avail) ? src + 4 * q + u : src, (u < avail) ? 4 : 0);
        }
    }
}

__device__ void lf_store_cols(const LeafArgs& a, const LfSmem& s, int64_t r0, int rows, int cbeg, int cend) {
    const int nq = (rows + 3) >> 2;
    const int total = (cend - cbeg) * nq;
    for (int e = threadIdx.x; e < total; e += LF_THREADS) {
        const int cc = cbeg + e / nq, q = e % nq;
        const float4 v = *reinterpret_cast<const float4*>(s.tile + (int64_t)cc * a.ldt + 4 * q);
        const int64_t gr = r0 + 4 * q;
        float* dq = a.Q + gr + (int64_t)cc * a.ldq;
        const float vv[4] = {v.x, v.y, v.z, v.w};
        ushort4 hb, lb;
        uint16_t* hbp = reinterpret_cast<uint16_t*>(&hb);
        uint16_t* lbp = reinterpret_cast<uint16_t*>(&lb);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            hbp[u] = lf_to16(vv[u], a.bf16);
            lbp[u] = lf_to16((vv[u] - lf_from16(hbp[u], a.bf16)) * 2048.f, a.bf16);
        }
        uint16_t* dh = a.Qh ? a.Qh + gr + (int64_t)cc * a.ldh : nullptr;
        uint16_t* dl = a.Ql ? a.Ql + gr + (int64_t)cc * a.ldh : nullptr;
        if (a.vec && 4 * q + 3 < rows) {
            __stcs(reinterpret_cast<float4*>(dq), v);
            if (dh) *reinterpret_cast<ushort4*>(dh) = hb;
            if (dl) *reinterpret_cast<ushort4*>(dl) = lb;
        } else {
#pragma unroll
            for (int u = 0; u < 4; ++u)
                if (4 * q + u < rows) {
                    dq[u] = vv[u];
                    if (dh) dh[u] = hbp[u];
                    if (dl) dl[u] = lbp[u];
                }
        }
    }
}

// R block output (CTA 0): rows [c0, c0 + 32) of the diagonal block from s.Racc, zero below.
__device__ void lf_write_r(const LeafArgs& a, const LfSmem& s, int c0, int ncp) {
    for (int e = threadIdx.x; e < ncp * ncp; e += LF_THREADS) {
        const int i = e % ncp, j = e / ncp;
        a.R[(c0 + i) + (int64_t)(c0 + j) * a.ldr] = (i <= j) ? (float)s.Racc[i * LF_GLD + j] : 0.f;
    }
}

// ------------------------------------------------------------------ the kernel
template <int NI>
__global__ void __launch_bounds__(LF_THREADS, 1) leaf_kernel(LeafArgs a) {
    extern __shared__ __align__(16) uint8_t lf_smem[];
    const LfSmem s(lf_smem, a.ldt);
    const int64_t r0 = (int64_t)blockIdx.x * a.rows_per;
    const int64_t rem = a.m - r0;
    const int rows = rem <= 0 ? 0 : (rem < a.rows_per ? (int)rem : a.rows_per);
    const int rp16 = (rows + 15) & ~15;
    const int h = a.nc < 32 ? a.nc : 32;
    const int w = a.nc - h;

    // rows of both panels in flight at once (two commit groups)
    lf_load_cols(a, s, r0, rows, rp16, 0, 32);
    lf_cp_commit();
    if (w > 0) lf_load_cols(a, s, r0, rows, rp16, 32, 64);
    lf_cp_commit();
    LF_MARK(0);
    lf_cp_wait<1>();
    __syncthreads();
    LF_MARK(1);

    // ---- panel 1
    int bad = lf_panel<NI>(a, s, 0, h, rp16, 2);
    if (bad >= 0) {
        if (blockIdx.x == 0 && threadIdx.x == 0) atomicMin(a.status, a.col0 + bad);
        return;   // uniform across the grid (every CTA factors the same reduced Gram)
    }
    if (blockIdx.x == 0) lf_write_r(a, s, 0, h);
    if (w > 0) {
        lf_cp_wait<0>();
        __syncthreads();
        // ---- R12 = Q1^T P2 and P2 -= Q1 R12
        LF_MARK(6);
        lf_k1(a, s, rp16);
        LF_MARK(7);
        lf_allreduce(a, s, 1024);
        LF_MARK(8);
        for (int e = threadIdx.x; e < 1024; e += LF_THREADS) {
            const int i = e >> 5, j = e & 31;   // R12(i, j)
            const float v = (i < h && j < w) ? (float)s.red[e] : 0.f;
            s.R12h[j * LF_R12LD + i] = lf_to16(-v, a.bf16);
            if (blockIdx.x == 0 && i < h && j < w) a.R[i + (int64_t)(h + j) * a.ldr] = v;
            if (blockIdx.x == 0 && i < w && j < h) a.R[(h + i) + (int64_t)j * a.ldr] = 0.f;
        }
        __syncthreads();
        lf_k2(a, s, rp16);
        LF_MARK(9);
        // Q1 is final: write it while panel 2 runs
        lf_store_cols(a, s, r0, rows, 0, h);
        LF_MARK(10);
        // ---- panel 2
        bad = lf_panel<NI>(a, s, 32, w, rp16, 11);
        if (bad >= 0) {
            if (blockIdx.x == 0 && threadIdx.x == 0) atomicMin(a.status, a.col0 + h + bad);
            return;
        }
        if (blockIdx.x == 0) {
            for (int e = threadIdx.x; e < w * w; e += LF_THREADS) {
                const int i = e % w, j = e / w;
                a.R[(h + i) + (int64_t)(h + j) * a.ldr] = (i <= j) ? (float)s.Racc[i * LF_GLD + j] : 0.f;
            }
        }
        LF_MARK(15);
        lf_store_cols(a, s, r0, rows, 32, 32 + w);
        LF_MARK(16);
    } else {
        lf_store_cols(a, s, r0, rows, 0, h);
    }
}

// ------------------------------------------------------------------ host side
static int lf_sms() {
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    return sms;
}
static int lf_smem_max() {
    static int v = 0;
    if (!v) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        v -= 1024;   // static shared memory + slack
    }
    return v;
}
static void lf_geometry(int64_t m, int& grid, int& rows_per, int& ldt) {
    grid = lf_sms() < LF_MAX_GRID ? lf_sms() : LF_MAX_GRID;
    rows_per = (int)(((m + grid - 1) / grid + 7) & ~int64_t(7));
    if (rows_per < 16) rows_per = 16;
    grid = (int)((m + rows_per - 1) / rows_per);
    if (grid < 1) grid = 1;
    const int rp16 = (rows_per + 15) & ~15;
    ldt = ((rp16 - 4 + 31) & ~31) + 4;   // == 4 mod 32, >= rp16
}

size_t leaf_smem_bytes(int64_t m) {
    int grid, rows_per, ldt;
    lf_geometry(m, grid, rows_per, ldt);
    return (size_t)64 * ldt * 4 + LfSmem::fixed_bytes();
}

bool leaf_fits(int64_t m) {
    if (getenv("RGSQR_NO_LEAF")) return false;
    int grid, rows_per, ldt;
    lf_geometry(m, grid, rows_per, ldt);
    return ((rows_per + 15) & ~15) <= 64 * LF_MAXI && leaf_smem_bytes(m) <= (size_t)lf_smem_max();
}

size_t leaf_ws_doubles() { return (size_t)(LF_MAX_GRID + 1) * LF_PART + 64; }

cudaError_t launch_leaf(const LeafLaunch& L, cudaStream_t st) {
    if (L.nc < 1 || L.nc > 64 || !leaf_fits(L.m)) return cudaErrorInvalidValue;
    LeafArgs a{};
    a.Q = L.Q;
    a.ldq = L.ldq;
    a.Qh = L.Qh;
    a.Ql = L.Ql;
    a.ldh = L.ldh;
    a.m = L.m;
    a.nc = L.nc;
    a.R = L.R;
    a.ldr = L.ldr;
    a.part = L.ws;
    a.red = L.ws + (size_t)LF_MAX_GRID * LF_PART;
    a.bar = L.bar;
    a.status = L.status;
    a.col0 = L.col0;
    a.bf16 = L.bf16;
    int grid;
    lf_geometry(L.m, grid, a.rows_per, a.ldt);
    a.vec = ((L.ldq & 3) == 0) && ((reinterpret_cast<uintptr_t>(L.Q) & 15) == 0) && ((L.ldh & 3) == 0) &&
            ((reinterpret_cast<uintptr_t>(L.Qh) & 7) == 0) && ((reinterpret_cast<uintptr_t>(L.Ql) & 7) == 0);
    const size_t smem = leaf_smem_bytes(L.m);
    const bool small = ((a.rows_per + 15) & ~15) <= 448;
    void (*kern)(LeafArgs) = small ? leaf_kernel<7> : leaf_kernel<LF_MAXI>;
    static size_t attr[2] = {0, 0};
    if (smem > attr[small]) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr[small] = smem;
    }
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(LF_THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeCooperative;   // co-residency for the grid barriers
    at[0].val.cooperative = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    ++g_launches;
    return cudaLaunchKernelEx(&cfg, kern, a);
}

}  // namespace rg
