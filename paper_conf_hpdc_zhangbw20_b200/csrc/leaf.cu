// leaf.cu -- the base case of Algorithm 1 in one kernel: the QR of a
// block of nc <= 64 columns (the leaf of the recursion, nb = 64; reading #2) by CholQR2 with an
// fp64 Gram matrix, optionally preceded by lines 8-9 of the level above (the "prologue"):
//
//   [prologue]  R_AB = Q_A^T P,  P <- P - Q_A R_AB     (16-bit operands, fp32 accumulation,
//                                                       the precision of the tensor-core GEMMs)
//   pass p:     G = P^T P (fp64),  R_p = chol(G),  P <- P R_p^{-1}
//   R = R_p ... R_1
//
// In exact arithmetic the leaf's Q and R are those of the two 32-column panels + K1 + K2 of the
// paper's structure (the QR of a full-rank block is unique), and the fp64 Gram makes the CholQR
// panel more accurate than the paper's fp32 MGS panel.  One CholQR pass when kappa_F(R_1) <= 2 nc
// (Q then orthogonal to ~kappa u32), else CholQR2; a failed pivot switches to shifted CholQR3
// (shift 11 (m nc + nc (nc + 1)) u ||P||_F^2); a pivot that still fails is a numerical breakdown
// reported through status (col0 + j).
//
// B200 design ("Leaf").  Every CTA of a cooperative grid (one per SM) owns a
// contiguous run of rows of the block, loads them once (cp.async) into shared memory and writes Q
// (fp32 + 16-bit shadow) once; a 65536 x 64 leaf is 16 MB, a few us of HBM traffic, so the kernel
// is latency-bound and built around few grid-wide steps:
//   * Gram on the fp64 tensor cores (DMMA m8n8k4) straight from the fp32 rows in smem (one
//     fragment per 8-column block serves as A and B), 36 8x8 blocks, no staging copy;
//   * one deterministic grid all-reduction per pass (fixed-order sums, two grid barriers);
//   * the 64 x 64 Cholesky on 4 warps (columns per lane, cyclic rows per warp, in registers), one
//     shared-memory row broadcast + producer/consumer named barrier per pivot; R^{-1} in fp32 by column-parallel back
//     substitution; P R^{-1} exploiting the triangle;
//   * the prologue on mma.sync m16n8k16 from a 16-bit staging copy of Q_A (replaces that level's
//     K1 GEMM, split-K reduce and K2 GEMM launches).
// Measured per-op (tools/prof_levels.py) and per-phase (tools/leaf_bench.cu) on B200.
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
constexpr int LF_GLD = 66;                   // fp64 64 x 64 matrices in smem: row stride (16-byte rows)
constexpr int LF_TLD = 68;                   // fp32 column-major R: column stride
constexpr int LF_NE = 64 * 65 / 2;           // packed upper-triangle Gram entries
constexpr int LF_NENT = 36 * 64;             // Gram fragment entries (36 8x8 blocks)
constexpr int LF_PART = 4096;                // doubles per CTA partial in the workspace (64 x 64 prologue)
constexpr int LF_ABLD = 72;                  // 16-bit -R_AB image [n][k] row stride (halves)
constexpr int LF_MAX_GRID = 160;
// Partial layout: entries in chunks of 8 consecutive doubles (64 B) per CTA, the CTAs' chunks of one
// entry range adjacent -- a CTA writes whole 64 B chunks, a reducing warp reads 32 CTAs x 64 B
// contiguously (one chunk = 8 entries per warp).
__host__ __device__ constexpr int64_t lf_pidx(int e, int b) {
    return (int64_t)(e >> 3) * (LF_MAX_GRID * 8) + b * 8 + (e & 7);
}
constexpr size_t LF_REGION = 33792;          // bytes of each of the two aliased scratch regions

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
    double* part;        // CTA partials in chunks of 8 entries: lf_pidx(e, b) (coalesced both ways)
    double* red;         // [LF_PART] reduced result
    double* racc;        // [2][64 * 64] accumulated R (CTA 0), row-major
    unsigned* bar;       // grid barrier word (generation bit flips every barrier)
    int* status;         // atomicMin(status, col0 + j) on a numerical breakdown
    int col0;
    int bf16;
    int rows_per;        // rows per CTA (multiple of 8)
    int ldt;             // smem tile leading dimension (floats), == 4 mod 32
    int vec;             // 16-byte global accesses allowed
    // prologue (Algorithm 1 lines 8-9 of the level above, folded in): R_AB = Q_A^T P, P -= Q_A R_AB
    const uint16_t* pq;  // Q_A, 16-bit image (ld ldh), m x ph; null: no prologue
    int ph;              // columns of Q_A (<= 64)
    int fast;            // first Gram on the 16-bit tensor cores (split fp16, see lf_gram16)
    int chol;            // fast-path Cholesky + inverse: 1 lf_chol_inv_b4 (default), 0 lf_chol_inv32
    unsigned long long* stats;   // [0] launches, [1] fast-Gram fallbacks, [2] CholQR passes (CTA 0)
};

// Per-handle counters (CTA 0, thread 0; read with RGSQR_LEAF_STATS=1): launches, fast-Gram
// fallbacks to the fp64 Gram, CholQR passes.
#define LF_COUNT(i, v)                                                        \
    do {                                                                      \
        if (blockIdx.x == 0 && threadIdx.x == 0) a.stats[(i) + 1] += (v);     \
    } while (0)
#ifdef LF_TRACE
__device__ unsigned long long lf_trace[48];
__device__ long long lf_clk[2];
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
        unsigned old;
        asm volatile("atom.add.release.gpu.global.u32 %0, [%1], %2;" : "=r"(old) : "l"(bar), "r"(nb) : "memory");
        while (((lf_ld_acquire(bar) ^ old) & 0x80000000u) == 0) {
        }
    }
    __syncthreads();
}

__device__ __forceinline__ void lf_bar128() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

__device__ __forceinline__ void lf_cp16(void* sdst, const void* gsrc, int src_bytes) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(sdst)), "l"(gsrc), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void lf_cp4(float* sdst, const float* gsrc, int src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(smem_u32(sdst)), "l"(gsrc), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void lf_cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void lf_cp_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

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

// fp64 1/sqrt: hardware approximation + one Newton step (relative error ~2^-44, far below what
// the fp32 outputs resolve; the pivot test is done on d itself).
__device__ __forceinline__ double lf_rsqrt(double d) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(d));
    const double e = fma(-d * y, y, 1.0);
    return fma(0.5 * y, e, y);
}

// ------------------------------------------------------------------ shared memory
// Regions A and B are adjacent and reused by phase:
//   A: Gram warp partials (scr) -> all-reduce result (red) -> fp32 R (Rt32) + R^{-1} (X32)
//   B: full Gram G -> R of the pass (Rs, fp64 row-major; written after every thread loaded G)
//   A + B: the prologue's 16-bit Q_A staging copy (qa)
struct LfSmem {
    float* tile;      // 64 columns x ldt rows (fp32, column-major)
    double* scr;      // A: LF_NENT doubles
    double* red;      // A: LF_NE doubles
    float* Rt32;      // A: 64 x LF_TLD, fp32 R column-major, R(i, j) = Rt32[j * LF_TLD + i]
    float* X32;       // A (+ Rt32 size): 64 x 64 fp32 R^{-1}, row-major
    double* G;        // B: 64 x LF_GLD full symmetric Gram
    double* Rs;       // B: 64 x LF_GLD R of the pass, row-major
    uint16_t* qa;     // A + B: prologue staging, 64 columns x lf_qa_ld halves
    double* U;        // 2 x 64: row k of the Schur complement (ping-pong)
    double* gdiag;    // 64: diagonal of G (pivot test)
    double* rdiag;    // 64: 1 / R(k, k)
    float* rdiag32;   // 64
    uint16_t* RABh;   // 64 x LF_ABLD: -R_AB as the prologue K2 B operand, [n][k]
    int* flag;        // 8 ints
    float* dsc;       // 64: 1 / (power-of-two column scale of X) in the tensor-core apply
    uint4* xfrag;     // 32 (k-step, n-tile) x 32 lanes: split fp16 B fragments of X = R^-1 (16 KB)
    static constexpr size_t fixed_bytes() {
        return 2 * LF_REGION + 2 * 64 * 8 + 64 * 8 + 64 * 8 + 64 * 4 + 64 * LF_ABLD * 2 + 64 + 64 * 4 + 16384;
    }
    __device__ LfSmem(uint8_t* base, int ldt) {
        tile = reinterpret_cast<float*>(base);
        uint8_t* p = base + (size_t)64 * ldt * 4;
        scr = reinterpret_cast<double*>(p);
        red = reinterpret_cast<double*>(p);
        Rt32 = reinterpret_cast<float*>(p);
        X32 = reinterpret_cast<float*>(p + 64 * LF_TLD * 4);
        qa = reinterpret_cast<uint16_t*>(p);
        p += LF_REGION;
        G = reinterpret_cast<double*>(p);
        Rs = reinterpret_cast<double*>(p);
        p += LF_REGION;
        U = reinterpret_cast<double*>(p);
        p += 2 * 64 * 8;
        gdiag = reinterpret_cast<double*>(p);
        p += 64 * 8;
        rdiag = reinterpret_cast<double*>(p);
        p += 64 * 8;
        rdiag32 = reinterpret_cast<float*>(p);
        p += 64 * 4;
        RABh = reinterpret_cast<uint16_t*>(p);
        p += 64 * LF_ABLD * 2;
        flag = reinterpret_cast<int*>(p);
        p += 64;
        dsc = reinterpret_cast<float*>(p);
        p += 64 * 4;
        xfrag = reinterpret_cast<uint4*>(p);
    }
};
static_assert(LF_NENT * 8 <= LF_REGION && LF_NE * 8 <= LF_REGION, "region A");
static_assert(64 * LF_TLD * 4 + 64 * 64 * 4 <= LF_REGION && 64 * LF_GLD * 8 <= LF_REGION, "regions");

__host__ __device__ __forceinline__ int lf_qa_ld(int rp16) { return ((rp16 - 8 + 63) & ~63) + 8; }   // == 8 mod 64 halves

// ------------------------------------------------------------------ grid all-reduction
// Sum of the CTA partials part[b][0, ne) (already written by this CTA) into a.red (and s.red).
// Deterministic: entry e is summed by one warp of CTA e / slice, lanes over CTAs lane, lane + 32,
// ... in order, then a fixed xor-shuffle tree.  Two grid barriers (measured ~1.6 us each with 148
// CTAs; per-CTA ready flags polled by many threads instead were ~3x slower -- L2 contention).
__device__ void lf_allreduce(const LeafArgs& a, const LfSmem& s, int ne, bool to_smem, int mk = 0) {
    lf_grid_sync(a.bar);
    if (mk) LF_MARK(mk);
    const int grid = gridDim.x;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nch = (ne + 7) >> 3;
    // chunk c is reduced by warp c / grid of CTA c % grid: lanes over CTAs lane, lane + 32, ... in
    // order, then a fixed xor-shuffle tree per entry (deterministic)
    for (int c = blockIdx.x + grid * warp; c < nch; c += grid * LF_NW) {
        constexpr int NB = (LF_MAX_GRID + 31) / 32;
        const double* src = a.part + (int64_t)c * (LF_MAX_GRID * 8);
        double2 p[NB][4];
#pragma unroll
        for (int u = 0; u < NB; ++u) {
            const int b = lane + 32 * u;
#pragma unroll
            for (int k = 0; k < 4; ++k)
                p[u][k] = b < grid ? __ldcg(reinterpret_cast<const double2*>(src + b * 8) + k) : make_double2(0.0, 0.0);
        }
        double sm[8];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            sm[2 * k] = p[0][k].x;
            sm[2 * k + 1] = p[0][k].y;
        }
#pragma unroll
        for (int u = 1; u < NB; ++u)
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                sm[2 * k] += p[u][k].x;
                sm[2 * k + 1] += p[u][k].y;
            }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1)
#pragma unroll
            for (int k = 0; k < 8; ++k) sm[k] += __shfl_xor_sync(0xffffffffu, sm[k], o);
        if (lane < 8) {
            double v = sm[0];
#pragma unroll
            for (int k = 1; k < 8; ++k) v = lane == k ? sm[k] : v;
            const int e = 8 * c + lane;
            if (e < ne) __stcg(a.red + e, v);
        }
    }
    if (mk) LF_MARK(mk + 1);
    lf_grid_sync(a.bar);
    if (mk) LF_MARK(mk + 2);
    if (!to_smem) return;
    // every thread's loads in flight at once (a load-then-store loop paid one L2 round trip per
    // iteration: ~1.4 us for the 2080-entry Gram)
    constexpr int MQ = (LF_PART + LF_THREADS - 1) / LF_THREADS;
    double v[MQ];
#pragma unroll
    for (int u = 0; u < MQ; ++u) {
        const int e = threadIdx.x + u * LF_THREADS;
        v[u] = e < ne ? __ldcg(a.red + e) : 0.0;
    }
#pragma unroll
    for (int u = 0; u < MQ; ++u) {
        const int e = threadIdx.x + u * LF_THREADS;
        if (e < ne) s.red[e] = v[u];
    }
    __syncthreads();
}

// ------------------------------------------------------------------ Gram (fp64 tensor cores)
// Block t = 0..35 enumerates (bi, bj), bi <= bj < 8, row by row; group q takes t = q, q + 4, ...
// (9 blocks); warp w = group (w & 3) x k-quarter (w >> 2).  The block indices must be compile-time
// (fragment registers), hence the template on the group.
__host__ __device__ constexpr int lf_blk_i(int t) {
    int bi = 0;
    while (t >= 8 - bi) {
        t -= 8 - bi;
        ++bi;
    }
    return bi;
}
__host__ __device__ constexpr int lf_blk_j(int t) {
    int bi = 0;
    while (t >= 8 - bi) {
        t -= 8 - bi;
        ++bi;
    }
    return bi + t;
}

template <int T>
__device__ __forceinline__ void lf_dmma_blk(double (&acc)[2], const double (&f)[8]) {
    constexpr int bi = lf_blk_i(T), bj = lf_blk_j(T);   // forced compile-time: f stays in registers
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(acc[0]), "+d"(acc[1])
                 : "d"(f[bi]), "d"(f[bj]));
}

template <int Q>
__device__ __forceinline__ void lf_gram_group(const LfSmem& s, int ldt, int rp, int kq, int lane, double (&acc)[9][2]) {
    const int g = lane >> 2, c = lane & 3;
    const float* col = s.tile + g * ldt + c;
#pragma unroll 1
    for (int k0 = 4 * kq; k0 < rp; k0 += 16) {
        double f[8];
#pragma unroll
        for (int b = 0; b < 8; ++b) f[b] = (double)col[8 * b * ldt + k0];
        lf_dmma_blk<Q + 0>(acc[0], f);
        lf_dmma_blk<Q + 4>(acc[1], f);
        lf_dmma_blk<Q + 8>(acc[2], f);
        lf_dmma_blk<Q + 12>(acc[3], f);
        lf_dmma_blk<Q + 16>(acc[4], f);
        lf_dmma_blk<Q + 20>(acc[5], f);
        lf_dmma_blk<Q + 24>(acc[6], f);
        lf_dmma_blk<Q + 28>(acc[7], f);
        lf_dmma_blk<Q + 32>(acc[8], f);
    }
}

// Partial G = P^T P of the CTA's rows [0, rp) (64 tile columns) -> packed upper triangle
// ([j (j + 1) / 2 + i]) in this CTA's workspace partial.
__device__ void lf_gram(const LeafArgs& a, const LfSmem& s, int rp) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int q = warp & 3, kq = warp >> 2;
    double acc[9][2];
#pragma unroll
    for (int u = 0; u < 9; ++u) acc[u][0] = acc[u][1] = 0.0;
    switch (q) {
        case 0: lf_gram_group<0>(s, a.ldt, rp, kq, lane, acc); break;
        case 1: lf_gram_group<1>(s, a.ldt, rp, kq, lane, acc); break;
        case 2: lf_gram_group<2>(s, a.ldt, rp, kq, lane, acc); break;
        default: lf_gram_group<3>(s, a.ldt, rp, kq, lane, acc); break;
    }
    // the four k-quarters summed in order through the scratch: entry e = ((q * 9 + u) * 2 + v) * 32 + ln
    constexpr int NQ = (LF_NENT + LF_THREADS - 1) / LF_THREADS;
    double run[NQ];
#pragma unroll
    for (int i = 0; i < NQ; ++i) run[i] = 0.0;
    for (int r = 0; r < 4; ++r) {
        __syncthreads();
        if (kq == r) {
            double* dst = s.scr + q * 9 * 64 + lane;
#pragma unroll
            for (int u = 0; u < 9; ++u) {
                dst[(2 * u) * 32] = acc[u][0];
                dst[(2 * u + 1) * 32] = acc[u][1];
            }
        }
        __syncthreads();
#pragma unroll
        for (int i = 0; i < NQ; ++i) {
            const int e = threadIdx.x + LF_THREADS * i;
            if (e < LF_NENT) run[i] += s.scr[e];
        }
    }
#pragma unroll
    for (int i = 0; i < NQ; ++i) {
        const int e = threadIdx.x + LF_THREADS * i;
        if (e < LF_NENT) {
            const int ln = e & 31, v = (e >> 5) & 1, qu = e >> 6, qq = qu / 9, u = qu % 9;
            const int t = qq + 4 * u;
            const int bi = lf_blk_i(t), bj = lf_blk_j(t);
            const int ii = 8 * bi + (ln >> 2), jj = 8 * bj + 2 * (ln & 3) + v;
            if (ii <= jj) __stcg(a.part + lf_pidx(jj * (jj + 1) / 2 + ii, blockIdx.x), run[i]);
        }
    }
}

// ------------------------------------------------------------------ Gram (16-bit tensor cores)
// G = P^T P from a two-term fp16 split of every entry x: hi = fp16(x), lo = fp16((x - hi) 2^11),
// x_i x_j = hi_i hi_j + 2^-11 (hi_i lo_j + lo_i hi_j) + O(2^-22 |x_i x_j|) -- three products on
// mma.sync m16n8k16 with fp32 accumulation (1024 FMA/clk/SM measured vs 64 for the fp64 DMMA of
// lf_gram).  The entries are the column-scaled (section 3.5, reading #4) and projected block:
// |x| <= 512, so nothing overflows fp16; a column whose norm has dropped below 0.01 (entries near
// the fp16 subnormal range) or any non-finite value sends the pass back to the fp64 Gram
// (lf_cholqr).  20 upper 16 x 8 tiles of the 64 x 64 Gram; warp = tile group q (5 tiles) x
// k-quarter kq; per element v = hh + 2^-11 mx in fp32, the four k-quarters summed in fixed
// order, stored as fp64 in the packed-upper-triangle partial of lf_gram.  Relative error ~1e-6
// of |P_i||P_j|: used for a single CholQR pass only when R is well conditioned (lf_cholqr).
__device__ __forceinline__ void lf_split2(float2 v, uint32_t& hi, uint32_t& lo) {
    const __half2 h = __floats2half2_rn(v.x, v.y);
    const float2 hf = __half22float2(h);
    const __half2 l = __floats2half2_rn((v.x - hf.x) * 2048.f, (v.y - hf.y) * 2048.f);
    hi = *reinterpret_cast<const uint32_t*>(&h);
    lo = *reinterpret_cast<const uint32_t*>(&l);
}

__device__ __forceinline__ void lf_mma_f16(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                           uint32_t b0, uint32_t b1) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// Tile groups (16 x 8 tiles (bi, cb): Gram rows 16 bi.., columns 8 cb..), chosen so that the work
// per k-step -- 3 mma per tile + one split of every 8-column block a tile touches -- is balanced:
//   q0: 16x16 blocks (0,0) (0,1) (1,1)  -> 6 tiles, column blocks 0-3
//   q1: 16x16 blocks (2,2) (2,3) (3,3)  -> 6 tiles, column blocks 4-7
//   q2: 16x16 blocks (0,2) (0,3)        -> 4 tiles, column blocks 0, 1, 4-7
//   q3: 16x16 blocks (1,2) (1,3)        -> 4 tiles, column blocks 2-7
__host__ __device__ constexpr int lf_t16_n(int q) { return q < 2 ? 6 : 4; }
__host__ __device__ constexpr int lf_t16_bi(int q, int t) {
    return q == 0 ? (t < 4 ? 0 : 1) : q == 1 ? (t < 4 ? 2 : 3) : q == 2 ? 0 : 1;
}
__host__ __device__ constexpr int lf_t16_cb(int q, int t) {
    return q == 0 ? (t < 4 ? t : t - 2) : q == 1 ? (t < 4 ? 4 + t : t + 2) : 4 + t;
}
__host__ __device__ constexpr bool lf_t16_need(int q, int cb) {
    bool need = false;
    for (int t = 0; t < lf_t16_n(q); ++t)
        need |= (lf_t16_cb(q, t) == cb) || (2 * lf_t16_bi(q, t) == cb) || (2 * lf_t16_bi(q, t) + 1 == cb);
    return need;
}

constexpr int LF_G16LD = 65;   // dense fp32 64 x 64 per k-quarter in the epilogue (odd: conflict-free)

// Partial Gram of the CTA's rows, group Q of k-quarter kq, written to the dense k-quarter slab.
template <int Q>
__device__ __forceinline__ void lf_gram16_group(const LfSmem& s, int ldt, int rp16, int kq, int lane, float* slab) {
    constexpr int NT = lf_t16_n(Q);
    const int g = lane >> 2, c = lane & 3;
    float hh[NT][4], mx[NT][4];
#pragma unroll
    for (int t = 0; t < NT; ++t)
#pragma unroll
        for (int u = 0; u < 4; ++u) hh[t][u] = mx[t][u] = 0.f;
#pragma unroll 1
    for (int k0 = 16 * kq; k0 < rp16; k0 += 64) {
        uint32_t fh[8][2], fl[8][2];
#pragma unroll
        for (int cb = 0; cb < 8; ++cb) {
            if (!lf_t16_need(Q, cb)) continue;   // compile-time: only the blocks this group's tiles touch
            const float* col = s.tile + (8 * cb + g) * ldt + k0 + 2 * c;
            lf_split2(*reinterpret_cast<const float2*>(col), fh[cb][0], fl[cb][0]);
            lf_split2(*reinterpret_cast<const float2*>(col + 8), fh[cb][1], fl[cb][1]);
        }
#pragma unroll
        for (int t = 0; t < NT; ++t) {
            const int bi = lf_t16_bi(Q, t), cb = lf_t16_cb(Q, t);
            const int r0 = 2 * bi, r1 = 2 * bi + 1;
            lf_mma_f16(hh[t], fh[r0][0], fh[r1][0], fh[r0][1], fh[r1][1], fh[cb][0], fh[cb][1]);
            lf_mma_f16(mx[t], fh[r0][0], fh[r1][0], fh[r0][1], fh[r1][1], fl[cb][0], fl[cb][1]);
            lf_mma_f16(mx[t], fl[r0][0], fl[r1][0], fl[r0][1], fl[r1][1], fh[cb][0], fh[cb][1]);
        }
    }
#pragma unroll
    for (int t = 0; t < NT; ++t) {
        const int bi = lf_t16_bi(Q, t), cb = lf_t16_cb(Q, t);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int i = 16 * bi + g + 8 * (u >> 1), j = 8 * cb + 2 * c + (u & 1);
            slab[i * LF_G16LD + j] = fmaf(mx[t][u], 0x1p-11f, hh[t][u]);
        }
    }
}

__device__ void lf_gram16(const LeafArgs& a, const LfSmem& s, int rp16) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int q = warp & 3, kq = warp >> 2;
    static_assert(4 * 64 * LF_G16LD * 4 <= 2 * LF_REGION, "scratch");   // regions A + B are adjacent
    float* slabs = reinterpret_cast<float*>(s.scr);
    float* slab = slabs + kq * 64 * LF_G16LD;
    switch (q) {
        case 0: lf_gram16_group<0>(s, a.ldt, rp16, kq, lane, slab); break;
        case 1: lf_gram16_group<1>(s, a.ldt, rp16, kq, lane, slab); break;
        case 2: lf_gram16_group<2>(s, a.ldt, rp16, kq, lane, slab); break;
        default: lf_gram16_group<3>(s, a.ldt, rp16, kq, lane, slab); break;
    }
    LF_MARK(25);
    __syncthreads();
    // the four k-quarters in fixed order -> fp64 packed upper triangle of the CTA partial
    // packed index p = j (j + 1) / 2 + i walked by consecutive threads: whole 64 B chunks per warp
#pragma unroll 2
    for (int p = threadIdx.x; p < LF_NE; p += LF_THREADS) {
        int j = (int)((sqrtf(8.f * (float)p + 1.f) - 1.f) * 0.5f);
        if ((j + 1) * (j + 2) / 2 <= p) ++j;
        if (j * (j + 1) / 2 > p) --j;
        const int i = p - j * (j + 1) / 2;
        const int o = i * LF_G16LD + j;
        constexpr int S = 64 * LF_G16LD;
        const float sum = ((slabs[o] + slabs[S + o]) + slabs[2 * S + o]) + slabs[3 * S + o];
        __stcg(a.part + lf_pidx(p, blockIdx.x), (double)sum);
    }
}

// ------------------------------------------------------------------ Cholesky (warps 0-3)
// s.G holds the full symmetric 64 x 64 Gram (identity beyond nc).  Warp q (< 4) keeps the rows
// i = 4 ii + q (ii < 16; cyclic, so the live rows stay balanced over the four SMSPs as the
// elimination proceeds) of the Schur complement S in registers, lane l columns l and l + 32.
// Step k (fully unrolled: k, and which register rows can still be live, are compile-time): the
// owner warp k % 4 has published S(k, :) (unnormalised) as row k of s.Rs; the three other warps
// wait for it on a producer/consumer named barrier (bar.arrive by the owner, bar.sync by the
// consumers, ids alternating 2 / 3), every thread forms t_j = S(k, j) / S(k, k) itself and updates
// its rows S(i, j) -= S(k, i) t_j.  The row that becomes pivot k + 1 is updated first and
// published at once (look-ahead), so the owner never waits.  Rows <= k are dead after
// publication and updated harmlessly; the columns < 32 are skipped once k >= 32.  The square
// roots, the pivot test and R(k, :) = S(k, :) / sqrt(S(k, k)) are done after the elimination.
// Measured on B200 (tools/leaf_bench.cu): 7.5 us per 64 x 64 factorization.  Slower variants: a
// barrier over all four warps per pivot with 16-row quarters per warp (11.2 us), one barrier per
// (consumer, owner) pair (7.7 us), permuted rows with all row loads issued up front (9.4 us), the
// whole 512-thread CTA, per-row mbarriers, one warp per 32 columns with shuffles, a fraction-free
// update.
// Writes s.Rs (fp64 row-major R, over G once every thread has loaded its part), s.Rt32 (fp32
// column-major), s.rdiag / s.rdiag32 (1 / R(k, k)).  Returns the first failed pivot (64 if none)
// on threads < 128: a pivot fails unless it is finite and > 1e-15 G(k, k).
__device__ __forceinline__ void lf_bar_sync(int id) { asm volatile("bar.sync %0, 128;" ::"r"(id) : "memory"); }
__device__ __forceinline__ void lf_bar_arrive(int id) { asm volatile("bar.arrive %0, 128;" ::"r"(id) : "memory"); }

// fp64 1/d: hardware approximation + one Newton step (relative error ~2^-44)
__device__ __forceinline__ double lf_rcp(double d) {
    double y;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(d));
    const double e = fma(-d, y, 1.0);
    return fma(y, e, y);
}

__device__ int lf_chol(const LfSmem& s) {
    const int t = threadIdx.x;   // < 128
    const int jl = t & 31, q = t >> 5;
    double g0[16], g1[16];
#pragma unroll
    for (int ii = 0; ii < 16; ++ii) {
        g0[ii] = s.G[(4 * ii + q) * LF_GLD + jl];
        g1[ii] = s.G[(4 * ii + q) * LF_GLD + jl + 32];
    }
    lf_bar128();   // every thread has its part of G before the rows overwrite it
    if (q == 0) {
        s.Rs[jl] = g0[0];
        s.Rs[jl + 32] = g1[0];
        __syncwarp();
        lf_bar_arrive(2);
    }
#pragma unroll
    for (int k = 0; k < 64; ++k) {
        const double* row = s.Rs + k * LF_GLD;
        if (q != (k & 3)) lf_bar_sync(2 + (k & 1));
        const double rd = lf_rcp(row[k]);
        const double t1 = (jl + 32 > k) ? row[jl + 32] * rd : 0.0;
        const double t0 = (k < 32 && jl > k) ? row[jl] * rd : 0.0;
        const int nx = (k + 1) >> 2;   // register row of pivot k + 1 in its owner warp
        if (k < 63) {
            const double v = row[4 * nx + q];
            g1[nx] = fma(-v, t1, g1[nx]);
            if (k < 32) g0[nx] = fma(-v, t0, g0[nx]);
            if (q == ((k + 1) & 3)) {
                double* nrow = s.Rs + (k + 1) * LF_GLD;
                if (k + 1 < 32) nrow[jl] = g0[nx];
                nrow[jl + 32] = g1[nx];
                __syncwarp();
                lf_bar_arrive(2 + ((k + 1) & 1));
            }
        }
#pragma unroll
        for (int ii = k >> 2; ii < 16; ++ii) {
            if (ii == nx && k < 63) continue;
            const double v = row[4 * ii + q];
            g1[ii] = fma(-v, t1, g1[ii]);
            if (k < 32) g0[ii] = fma(-v, t0, g0[ii]);
        }
    }
    lf_bar128();
    // pivots -> 1 / R(k, k) and the pivot test; then R(k, j) = S(k, j) / sqrt(S(k, k)), j >= k
    __shared__ int s_bad[2];
    if (t < 64) {
        const double d = s.Rs[t * LF_GLD + t];
        const bool good = (d > s.gdiag[t] * 1e-15) && isfinite(d);
        const double rs = good ? lf_rsqrt(d) : 1.0;
        s.rdiag[t] = rs;
        s.rdiag32[t] = (float)rs;
        const unsigned badm = __ballot_sync(0xffffffffu, !good);
        if (jl == 0) s_bad[t >> 5] = badm ? (__ffs(badm) - 1 + 32 * (t >> 5)) : 64;
    }
    lf_bar128();
    for (int e = t; e < 64 * 64; e += 128) {
        const int i = e >> 6, j = e & 63;
        const double r = (j >= i) ? s.Rs[i * LF_GLD + j] * s.rdiag[i] : 0.0;
        s.Rs[i * LF_GLD + j] = r;
        s.Rt32[j * LF_TLD + i] = (float)r;
    }
    lf_bar128();
    return min(s_bad[0], s_bad[1]);
}

// Fast path (after the split Gram): Cholesky AND inverse in one pivot loop, fp32.  The elimination
// of lf_chol (warps 0-3, rows 4 ii + q in registers, pivot rows published through shared memory
// with producer / consumer named barriers, look-ahead on row k + 1) is applied to the augmented
// [S | W] with W = I: after step k, S = U = L^{-1} G (upper) and W = L^{-1} (unit lower), G = L D L^T,
// so R = D^{-1/2} U and R^{-1} = W^T D^{-1/2} come out together -- the separate blocked inverse
// (lf_inverse) leaves the critical path.  fp32 is enough here: the split Gram carries ~1e-6
// relative error and the fast path is taken only for kappa_F(equilibrated) <= 1.1 nc.
// Writes s.X32 = R^{-1} (row-major), s.Rs = R (fp64 row-major, for the output / racc),
// s.rdiag32; *keq = kappa_F^2 of the column-equilibrated block.  Returns the first failed pivot
// (64 if none): a pivot fails unless finite and > 1e-4 G(k, k) (beyond that kappa, the fp64
// path takes over anyway).  Called by all threads.
constexpr int LF_PUB = 129;   // published rows: S (0..63) | W (64..127), odd stride
#ifndef LF_CHOL_WARPS
#define LF_CHOL_WARPS 16
#endif
#ifndef LF_CHOL_BLOCKED
#define LF_CHOL_BLOCKED 1   // 1: 4 x 4-block LDL (lf_chol_inv_b4); 0: the 64-pivot loop (lf_chol_inv32)
#endif

__device__ __forceinline__ float lf_rcp32(float x) {
    float y;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

template <int CW>   // warps in the elimination (rows 4 ii + q for CW = 4, CW ii + q in general)
__device__ int lf_chol_inv32(const LfSmem& s, int nc, double* keq) {
    static_assert(64 * LF_PUB * 4 <= LF_REGION, "region B");
    static_assert(CW == 4 || CW == 8 || CW == 16, "elimination warps");
    constexpr int RPW = 64 / CW;        // register rows per warp
    constexpr int NT = 32 * CW;         // named-barrier thread count
    float* pub = reinterpret_cast<float*>(s.G);
    const int t = threadIdx.x, jl = t & 31, q = t >> 5;
    __shared__ int s_bad2[2];
    __shared__ double s_en[LF_NW];
    auto bsync = [&](int id) { asm volatile("bar.sync %0, %1;" ::"r"(id), "n"(NT) : "memory"); };
    auto barrive = [&](int id) { asm volatile("bar.arrive %0, %1;" ::"r"(id), "n"(NT) : "memory"); };
    if (t < NT) {
        float g0[RPW], g1[RPW], w0[RPW], w1[RPW];
#pragma unroll
        for (int ii = 0; ii < RPW; ++ii) {
            const int i = CW * ii + q;
            g0[ii] = (float)s.G[i * LF_GLD + jl];
            g1[ii] = (float)s.G[i * LF_GLD + jl + 32];
            w0[ii] = (i == jl) ? 1.f : 0.f;
            w1[ii] = (i == jl + 32) ? 1.f : 0.f;
        }
        bsync(1);   // every thread has its part of G before the rows overwrite it
        if (q == 0) {
            pub[jl] = g0[0];
            pub[jl + 32] = g1[0];
            pub[64 + jl] = w0[0];
            pub[96 + jl] = w1[0];
            __syncwarp();
            barrive(2);
        }
#pragma unroll
        for (int k = 0; k < 64; ++k) {
            const float* row = pub + k * LF_PUB;
            if (q != (k % CW)) bsync(2 + (k & 1));
            const float rd = lf_rcp32(row[k]);
            const float t1 = (jl + 32 > k) ? row[jl + 32] * rd : 0.f;
            const float t0 = (k < 32 && jl > k) ? row[jl] * rd : 0.f;
            const float u0 = (jl <= k) ? row[64 + jl] * rd : 0.f;
            const float u1 = (k >= 32 && jl + 32 <= k) ? row[96 + jl] * rd : 0.f;
            const int nx = (k + 1) / CW;   // register row of pivot k + 1 in its owner warp
            if (k < 63) {
                const float v = row[CW * nx + q];
                g1[nx] = fmaf(-v, t1, g1[nx]);
                if (k < 32) g0[nx] = fmaf(-v, t0, g0[nx]);
                w0[nx] = fmaf(-v, u0, w0[nx]);
                if (k >= 32) w1[nx] = fmaf(-v, u1, w1[nx]);
                if (q == ((k + 1) % CW)) {
                    float* nrow = pub + (k + 1) * LF_PUB;
                    if (k + 1 < 32) nrow[jl] = g0[nx];
                    nrow[jl + 32] = g1[nx];
                    nrow[64 + jl] = w0[nx];
                    nrow[96 + jl] = w1[nx];
                    __syncwarp();
                    barrive(2 + ((k + 1) & 1));
                }
            }
#pragma unroll
            for (int ii = k / CW; ii < RPW; ++ii) {
                if (ii == nx && k < 63) continue;
                const float v = row[CW * ii + q];
                g1[ii] = fmaf(-v, t1, g1[ii]);
                if (k < 32) g0[ii] = fmaf(-v, t0, g0[ii]);
                w0[ii] = fmaf(-v, u0, w0[ii]);
                if (k >= 32) w1[ii] = fmaf(-v, u1, w1[ii]);
            }
        }
    }
    __syncthreads();
    LF_MARK(28);
    if (t < 64) {
        const float d = pub[t * LF_PUB + t];
        const bool good = (d > (float)s.gdiag[t] * 1e-4f) && isfinite(d);
        s.rdiag32[t] = good ? rsqrtf(d) : 1.f;
        const unsigned badm = __ballot_sync(0xffffffffu, !good);
        if (jl == 0) s_bad2[t >> 5] = badm ? (__ffs(badm) - 1 + 32 * (t >> 5)) : 64;
    }
    __syncthreads();
    // X(i, j) = W(j, i) / sqrt(d_j) (i <= j),  R(i, j) = U(i, j) / sqrt(d_i) (j >= i)
    constexpr int PER = 64 * 64 / LF_THREADS;
    float rr[PER];
    double en = 0.0;
#pragma unroll
    for (int u = 0; u < PER; ++u) {
        const int e = t + u * LF_THREADS, i = e >> 6, j = e & 63;
        const float x = (i <= j) ? pub[j * LF_PUB + 64 + i] * s.rdiag32[j] : 0.f;
        s.X32[e] = x;
        rr[u] = (j >= i) ? pub[i * LF_PUB + j] * s.rdiag32[i] : 0.f;
        if (i < nc && j < nc && i <= j) en = fma((double)x * x, s.gdiag[i], en);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) en += __shfl_xor_sync(0xffffffffu, en, o);
    if (jl == 0) s_en[t >> 5] = en;
    __syncthreads();   // pub (region B) fully read: R may overwrite it
    double se = 0.0;
#pragma unroll
    for (int w = 0; w < LF_NW; ++w) se += s_en[w];
    *keq = (double)nc * se;
#pragma unroll
    for (int u = 0; u < PER; ++u) {
        const int e = t + u * LF_THREADS, i = e >> 6, j = e & 63;
        s.Rs[i * LF_GLD + j] = (double)rr[u];
    }
    __syncthreads();
    return min(s_bad2[0], s_bad2[1]);
}

// Fast path, 4 x 4-block form: G = L_b D_b L_b^T with 4 x 4 diagonal blocks, 16 block steps instead
// of 64 pivots.  Four warps, lane = one column: warp 0 G(:, 0..31), warp 1 G(:, 32..63), warp 2
// W(:, 0..31), warp 3 W(:, 32..63) (W = L_b^-1, starting from I).  Block step K (rows / columns
// 4K..4K+3), every lane:
//   A_KK  <- the 4 x 4 pivot block (published by the G lanes, 4 floats per column, one STS.128)
//   R_KK  = chol(A_KK) in registers (every lane redundantly: 4 rsqrt on the chain)
//   z     = R_KK^-T x_K,  y = R_KK^-1 z       (x_K: the lane's column at rows 4K..4K+3)
//   x_i  -= A(i, 4K..4K+3) y  for the trailing rows i
// so one publish + one named barrier + a 4 x 4 factorisation per FOUR pivots.  z is final output:
// for a G column it is R(4K..4K+3, col); for a W column it is X(col, 4K..4K+3) (R = R_D L_b^T,
// X = R^-1 = W^T R_D^-1).  The columns are kept rotated (x[0..3] = rows 4K..4K+3), the steps run in
// rolled loops, and the register length shrinks by 16 every 4 steps (only the live rows are
// updated).  Measured (tools/leaf_bench.cu, ncu source view): a fully unrolled 32- or 64-step pivot
// chain is ~25 KB of straight-line SASS executed once per launch and stalls on instruction fetch
// (77 % stall_no_instruction); a one-warp register LDL with shuffles or a shared-memory row
// broadcast costs 120-175 cycles per pivot even when the code is cached, so 64 single pivots stay
// >= 4 us -- the 4 x 4 blocks cut the dependent steps to 16.  In the pipeline the variants are
// within 1 % of each other (RGSQR_LEAF_CHOL=0 selects the 64-pivot loop): the leaf is bound by
// its cold-code / cold-data phases, not by this factorisation.
constexpr int LF_B4ROWS = 80;   // rows per publish buffer (4K + L - 1 <= 75: tail reads are garbage-in, unused)
constexpr int LF_RST = 65;      // fp32 R scratch row stride

struct LfB4 {
    float4* buf;    // 2 x LF_B4ROWS: buf[(K & 1) * LF_B4ROWS + col] = rows 4K..4K+3 of column col
    float* Rst;     // 64 x LF_RST fp32 R (row-major, upper valid)
    float* XT;      // 64 x 64: XT[a * 64 + b] = X(b, a)
    float* sd;      // 64 pivots d
    float* srd;     // 64: 1 / R(k, k)
};

// Steps K0 .. K0+3 on a column of register length L (x[p] = row 4K + p).  PUB: publish x[0..3] at
// column col; GCOL: z goes to R (else to X^T); REC: record pivots / 1 / R(k, k).
template <int L, bool PUB, bool GCOL, bool REC>
__device__ __forceinline__ void lf_b4_phase(float (&x)[64], int K0, int col, int lane, const LfB4& b) {
#pragma unroll 1
    for (int K = K0; K < K0 + 4; ++K) {
        float4* bk = b.buf + (K & 1) * LF_B4ROWS;
        if (PUB) bk[col] = make_float4(x[0], x[1], x[2], x[3]);
        asm volatile("bar.sync 8, 128;" ::: "memory");
        const int k0 = 4 * K;
        const float4 c0 = bk[k0], c1 = bk[k0 + 1], c2 = bk[k0 + 2], c3 = bk[k0 + 3];
        // R_KK = chol(A_KK), A(r, c) (r <= c) = component r of column 4K + c
        const float d0 = c0.x, i0 = rsqrtf(d0);
        const float r01 = c1.x * i0, r02 = c2.x * i0, r03 = c3.x * i0;
        const float d1 = fmaf(-r01, r01, c1.y), i1 = rsqrtf(d1);
        const float r12 = fmaf(-r01, r02, c2.y) * i1, r13 = fmaf(-r01, r03, c3.y) * i1;
        const float d2 = fmaf(-r12, r12, fmaf(-r02, r02, c2.z)), i2 = rsqrtf(d2);
        const float r23 = fmaf(-r12, r13, fmaf(-r02, r03, c3.z)) * i2;
        const float d3 = fmaf(-r23, r23, fmaf(-r13, r13, fmaf(-r03, r03, c3.w))), i3 = rsqrtf(d3);
        // z = R_KK^-T x_K, y = R_KK^-1 z
        const float z0 = x[0] * i0;
        const float z1 = fmaf(-r01, z0, x[1]) * i1;
        const float z2 = fmaf(-r12, z1, fmaf(-r02, z0, x[2])) * i2;
        const float z3 = fmaf(-r23, z2, fmaf(-r13, z1, fmaf(-r03, z0, x[3]))) * i3;
        const float y3 = z3 * i3;
        const float y2 = fmaf(-r23, y3, z2) * i2;
        const float y1 = fmaf(-r13, y3, fmaf(-r12, y2, z1)) * i1;
        const float y0 = fmaf(-r03, y3, fmaf(-r02, y2, fmaf(-r01, y1, z0))) * i0;
        if (GCOL) {
            b.Rst[(k0 + 0) * LF_RST + col] = z0;
            b.Rst[(k0 + 1) * LF_RST + col] = z1;
            b.Rst[(k0 + 2) * LF_RST + col] = z2;
            b.Rst[(k0 + 3) * LF_RST + col] = z3;
        } else {
            b.XT[(k0 + 0) * 64 + col] = z0;
            b.XT[(k0 + 1) * 64 + col] = z1;
            b.XT[(k0 + 2) * 64 + col] = z2;
            b.XT[(k0 + 3) * 64 + col] = z3;
        }
        if (REC && lane == 0) {
            b.sd[k0] = d0, b.sd[k0 + 1] = d1, b.sd[k0 + 2] = d2, b.sd[k0 + 3] = d3;
            b.srd[k0] = i0, b.srd[k0 + 1] = i1, b.srd[k0 + 2] = i2, b.srd[k0 + 3] = i3;
        }
        // trailing rows: x[p - 4] = x[p] - A(4K + p, 4K..4K+3) y
#pragma unroll
        for (int p = 4; p < L; ++p) {
            const float4 v = bk[k0 + p];
            x[p - 4] = fmaf(-v.w, y3, fmaf(-v.z, y2, fmaf(-v.y, y1, fmaf(-v.x, y0, x[p]))));
        }
#pragma unroll
        for (int p = L - 4; p < L; ++p) x[p] = 0.f;
    }
}

template <int L>
__device__ __forceinline__ void lf_b4_idle(int K0) {
#pragma unroll 1
    for (int K = K0; K < K0 + 4; ++K) asm volatile("bar.sync 8, 128;" ::: "memory");
}

__device__ int lf_chol_inv_b4(const LfSmem& s, int nc, double* keq) {
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    float* G32 = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(s.red) + LF_NE * 8);   // region A, after red
    static_assert(LF_NE * 8 + 64 * LF_RST * 4 <= LF_REGION, "region A: red + G32");
    static_assert(64 * 64 * 4 <= LF_NE * 8, "region A: X^T over red");
    LfB4 b;
    b.buf = reinterpret_cast<float4*>(s.G);
    b.Rst = reinterpret_cast<float*>(b.buf + 2 * LF_B4ROWS);
    static_assert(2 * LF_B4ROWS * 16 + 64 * LF_RST * 4 <= LF_REGION, "region B");
    b.XT = reinterpret_cast<float*>(s.red);
    __shared__ float s_d[64], s_rd[64];
    __shared__ double s_en[LF_NW];
    __shared__ int s_bad3[2];
    b.sd = s_d;
    b.srd = s_rd;
    // dense fp32 G (identity beyond nc)
#pragma unroll
    for (int u = 0; u < 64 * 64 / LF_THREADS; ++u) {
        const int e = t + u * LF_THREADS, i = e >> 6, j = e & 63;
        const int lo = min(i, j), hi = max(i, j);
        G32[i * LF_RST + j] = (hi < nc) ? (float)s.red[hi * (hi + 1) / 2 + lo] : (i == j ? 1.f : 0.f);
    }
    __syncthreads();   // s.red dead: X^T may overwrite it
    if (warp < 4) {
        float x[64];
        if (warp == 0) {          // G(:, 0..31): rows 0..31, steps 0..7
#pragma unroll
            for (int p = 0; p < 32; ++p) x[p] = G32[p * LF_RST + lane];
            lf_b4_phase<32, true, true, false>(x, 0, lane, lane, b);
            lf_b4_phase<16, true, true, false>(x, 4, lane, lane, b);
            lf_b4_idle<0>(8);
            lf_b4_idle<0>(12);
        } else if (warp == 1) {   // G(:, 32..63): all rows, all steps
#pragma unroll
            for (int p = 0; p < 64; ++p) x[p] = G32[p * LF_RST + 32 + lane];
            lf_b4_phase<64, true, true, true>(x, 0, 32 + lane, lane, b);
            lf_b4_phase<48, true, true, true>(x, 4, 32 + lane, lane, b);
            lf_b4_phase<32, true, true, true>(x, 8, 32 + lane, lane, b);
            lf_b4_phase<16, true, true, true>(x, 12, 32 + lane, lane, b);
        } else if (warp == 2) {   // W(:, 0..31) from I
#pragma unroll
            for (int p = 0; p < 64; ++p) x[p] = (p == lane) ? 1.f : 0.f;
            lf_b4_phase<64, false, false, false>(x, 0, lane, lane, b);
            lf_b4_phase<48, false, false, false>(x, 4, lane, lane, b);
            lf_b4_phase<32, false, false, false>(x, 8, lane, lane, b);
            lf_b4_phase<16, false, false, false>(x, 12, lane, lane, b);
        } else {                  // W(:, 32..63): zero above row 32 (steps 0..7 are no-ops)
#pragma unroll
            for (int p = 0; p < 32; ++p) x[p] = (p == lane) ? 1.f : 0.f;   // rows 32.. after 8 steps
            lf_b4_idle<0>(0);
            lf_b4_idle<0>(4);
            lf_b4_phase<32, false, false, false>(x, 8, 32 + lane, lane, b);
            lf_b4_phase<16, false, false, false>(x, 12, 32 + lane, lane, b);
            // X(32 + lane, 0..31) = 0 (W(0..31, 32 + lane) = 0): not written by the steps
#pragma unroll 4
            for (int a = 0; a < 32; ++a) b.XT[a * 64 + 32 + lane] = 0.f;
        }
    }
    __syncthreads();
    LF_MARK(28);
    // X (row-major) from X^T, kappa term, R -> registers
    constexpr int PER = 64 * 64 / LF_THREADS;
    double en = 0.0;
    float rr[PER];
#pragma unroll
    for (int u = 0; u < PER; ++u) {
        const int e = t + u * LF_THREADS, i = e >> 6, j = e & 63;
        const float x = (i <= j) ? b.XT[j * 64 + i] : 0.f;
        s.X32[e] = x;
        rr[u] = (i <= j) ? b.Rst[i * LF_RST + j] : 0.f;
        if (i <= j && j < nc) en = fma((double)x * x, s.gdiag[i], en);
    }
    if (t < 64) {
        const float d = s_d[t];
        const bool good = (d > (float)s.gdiag[t] * 1e-4f) && isfinite(d);
        s.rdiag32[t] = s_rd[t];
        const unsigned badm = __ballot_sync(0xffffffffu, !good);
        if (lane == 0) s_bad3[warp] = badm ? (__ffs(badm) - 1 + 32 * warp) : 64;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) en += __shfl_xor_sync(0xffffffffu, en, o);
    if (lane == 0) s_en[warp] = en;
    __syncthreads();   // scratch fully read: s.Rs (region B) may overwrite it
    double se = 0.0;
#pragma unroll
    for (int w = 0; w < LF_NW; ++w) se += s_en[w];
    *keq = (double)nc * se;
#pragma unroll
    for (int u = 0; u < PER; ++u) {
        const int e = t + u * LF_THREADS, i = e >> 6, j = e & 63;
        s.Rs[i * LF_GLD + j] = (double)rr[u];
    }
    const int bad = min(s_bad3[0], s_bad3[1]);
    __syncthreads();
    return bad;
}

// X = R^{-1} (upper, fp32: it only feeds the fp32 product P R^{-1} and the kappa test), blocked
// on 32 x 32 blocks, whole CTA:
//   X11 = R11^{-1}, X22 = R22^{-1}   threads 0..63, column-parallel back substitution (right-
//                                    looking: each step one multiply + independent FMAs)
//   T   = R12 X22,  X12 = -X11 T     all threads, 1024 outputs each
// Writes s.X32 (row-major) and returns |R|_F^2 |R^{-1}|_F^2 over the nc x nc block (all threads).
__device__ double lf_inverse(const LfSmem& s, int nc, double* keq = nullptr) {
    const int tid = threadIdx.x;
    __shared__ double s_norm[3][LF_NW];
    if (tid < 64) {
        const int base = tid < 32 ? 0 : 32, j = tid & 31;
        float b[32];
#pragma unroll
        for (int i = 0; i < 32; ++i) b[i] = (i == j) ? 1.f : 0.f;
#pragma unroll
        for (int k = 31; k >= 0; --k) {
            b[k] *= s.rdiag32[base + k];
            const float* col = s.Rt32 + (base + k) * LF_TLD + base;
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
#pragma unroll
        for (int i = 0; i < 32; ++i) s.X32[(base + i) * 64 + base + j] = b[i];
    }
    __syncthreads();
    // T = R12 X22 into the X21 slot (rows 32.., cols 0..31: zero afterwards).  The 32-term dots are
    // fully unrolled over k with the triangle as predication (X22 is upper: X22(k, jj) = 0 for
    // k > jj, stored as zero), so all loads issue back to back and four FMA chains interleave (a
    // runtime-bounded loop waited on every shared load: ~1 us per product).
    float tv[2];
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int e = tid + LF_THREADS * q, i = e >> 5, jj = e & 31;
        float a4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int k = 0; k < 32; ++k)
            a4[k & 3] = fmaf(s.Rt32[(32 + k) * LF_TLD + i], s.X32[(32 + k) * 64 + 32 + jj], a4[k & 3]);
        tv[q] = (a4[0] + a4[1]) + (a4[2] + a4[3]);
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int e = tid + LF_THREADS * q, i = e >> 5, jj = e & 31;
        s.X32[(32 + i) * 64 + jj] = tv[q];
    }
    __syncthreads();
    // X12 = -X11 T (X11 upper: X11(i, k) = 0 for k < i, stored as zero; unrolled as above)
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int e = tid + LF_THREADS * q, i = e >> 5, jj = e & 31;
        float a4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int k = 0; k < 32; ++k) a4[k & 3] = fmaf(s.X32[i * 64 + k], s.X32[(32 + k) * 64 + jj], a4[k & 3]);
        tv[q] = -((a4[0] + a4[1]) + (a4[2] + a4[3]));
    }
    __syncthreads();
    double xn = 0.0, rn = 0.0, en = 0.0;
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int e = tid + LF_THREADS * q, i = e >> 5, jj = e & 31;
        s.X32[i * 64 + 32 + jj] = tv[q];
        s.X32[(32 + i) * 64 + jj] = 0.f;
    }
    __syncthreads();
    for (int e = tid; e < 64 * 64; e += LF_THREADS) {
        const int i = e >> 6, jj = e & 63;
        if (i < nc && jj < nc && i <= jj) {   // the identity padding beyond nc is not part of the block
            const double x = s.X32[e], r = s.Rs[i * LF_GLD + jj];
            xn = fma(x, x, xn);
            rn = fma(r, r, rn);
            en = fma(x * x, s.gdiag[i], en);   // (|p_i| X_ij)^2: R^-1 of the column-equilibrated block
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        xn += __shfl_xor_sync(0xffffffffu, xn, o);
        rn += __shfl_xor_sync(0xffffffffu, rn, o);
        en += __shfl_xor_sync(0xffffffffu, en, o);
    }
    if ((tid & 31) == 0) {
        s_norm[0][tid >> 5] = xn;
        s_norm[1][tid >> 5] = rn;
        s_norm[2][tid >> 5] = en;
    }
    __syncthreads();
    double sx = 0.0, sr = 0.0, se = 0.0;
#pragma unroll
    for (int w = 0; w < LF_NW; ++w) {
        sx += s_norm[0][w];
        sr += s_norm[1][w];
        se += s_norm[2][w];
    }
    // kappa_F^2 of the column-equilibrated block R D^-1 (D = diag |p_j|): |R D^-1|_F^2 = nc
    if (keq) *keq = (double)nc * se;
    return sx * sr;
}

// tile rows [0, rp) <- tile * R^{-1} (fp32).  Warp w takes the column group cg = w % 8 (8
// columns) and the rows (w / 8) * 32 + lane + 64 i (i < NI); R^{-1} is upper, so the k loop stops
// at the group's last column (warp-uniform).
template <int NI>
__device__ void lf_apply(const LeafArgs& a, const LfSmem& s, int rp) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // warps w, w + 4, w + 8, w + 12 share an SMSP: give them column groups s, 7 - s, s, 7 - s
    // (equal triangle work per SMSP)
    const int sp = warp & 3, t4 = warp >> 2;
    const int cg = (t4 & 1) ? 7 - sp : sp, half = t4 >> 1;
    const int ld = a.ldt;
    const int r0 = half * 32 + lane;
    float o[NI][8];
#pragma unroll
    for (int i = 0; i < NI; ++i)
#pragma unroll
        for (int c = 0; c < 8; ++c) o[i][c] = 0.f;
    const float* base = s.tile + r0;
    const int kend = 8 * cg + 8;
    int off = 0;
#pragma unroll 2
    for (int k = 0; k < kend; ++k, off += ld) {
        const float4 x0 = *reinterpret_cast<const float4*>(s.X32 + k * 64 + 8 * cg);
        const float4 x1 = *reinterpret_cast<const float4*>(s.X32 + k * 64 + 8 * cg + 4);
#pragma unroll
        for (int i = 0; i < NI; ++i) {
            const float x = base[off + 64 * i];   // rows >= rp: zeros or unused
            o[i][0] = fmaf(x, x0.x, o[i][0]);
            o[i][1] = fmaf(x, x0.y, o[i][1]);
            o[i][2] = fmaf(x, x0.z, o[i][2]);
            o[i][3] = fmaf(x, x0.w, o[i][3]);
            o[i][4] = fmaf(x, x1.x, o[i][4]);
            o[i][5] = fmaf(x, x1.y, o[i][5]);
            o[i][6] = fmaf(x, x1.z, o[i][6]);
            o[i][7] = fmaf(x, x1.w, o[i][7]);
        }
    }
    __syncthreads();
    float* ob = s.tile + 8 * cg * ld + r0;
#pragma unroll
    for (int i = 0; i < NI; ++i)
        if (r0 + 64 * i < rp)
#pragma unroll
            for (int c = 0; c < 8; ++c) ob[c * ld + 64 * i] = o[i][c];
    __syncthreads();
}

// tile rows [0, rp) <- tile * R^{-1} on the 16-bit tensor cores (fast path only): Q = P X with the
// two-term fp16 split of both operands, Q ~ Ph Xh + 2^-11 (Ph Xl + Pl Xh) (mma.sync m16n8k16, fp32
// accumulation; relative error ~1e-6 like the split Gram).  X's columns carry power-of-two scales
// c_j (largest |X_ij c_j| in [2^7, 2^8)), undone exactly on the output.  X is pre-split once into
// fragment-ordered hi/lo B operands (s.xfrag); warp w owns the 16-row blocks w, w + 16, .. and
// computes all 64 output columns of them (only the k-steps ks <= nt / 2 the triangle needs), so
// it reads and overwrites only its own rows: no block-wide barrier inside.
__device__ void lf_apply16(const LeafArgs& a, const LfSmem& s, int rp16) {
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int g = lane >> 2, c = lane & 3;
    if (tid < 64) {   // column scales of X (upper triangular: rows 0..j)
        float mx = 0.f;
        for (int k = 0; k <= tid; ++k) mx = fmaxf(mx, fabsf(s.X32[k * 64 + tid]));
        int e = 0;
        if (mx > 0.f) frexpf(mx, &e);
        const int ex = min(120, max(-120, 8 - e));
        s.dsc[tid] = ldexpf(1.f, -ex);                       // 1 / c_j
        reinterpret_cast<float*>(s.U)[tid] = ldexpf(1.f, ex);   // c_j (scratch)
    }
    __syncthreads();
    const float* cs = reinterpret_cast<const float*>(s.U);
    for (int e = tid; e < 32 * 32; e += LF_THREADS) {
        const int pi = e >> 5, ln = e & 31, ks = pi >> 3, nt = pi & 7;
        const int gg = ln >> 2, cc = ln & 3;
        const int n = 8 * nt + gg;
        const float sc = cs[n];
        const int k0 = 16 * ks + 2 * cc;
        const float2 v0 = make_float2(s.X32[k0 * 64 + n] * sc, s.X32[(k0 + 1) * 64 + n] * sc);
        const float2 v1 = make_float2(s.X32[(k0 + 8) * 64 + n] * sc, s.X32[(k0 + 9) * 64 + n] * sc);
        uint4 f;
        lf_split2(v0, f.x, f.z);
        lf_split2(v1, f.y, f.w);
        s.xfrag[e] = f;   // {hi b0, hi b1, lo b0, lo b1}
    }
    __syncthreads();
    const int ld = a.ldt;
    for (int rb = warp; 16 * rb < rp16; rb += LF_NW) {
        const int r0 = 16 * rb;
        float hh[8][4], mx[8][4];
#pragma unroll
        for (int nt = 0; nt < 8; ++nt)
#pragma unroll
            for (int u = 0; u < 4; ++u) hh[nt][u] = mx[nt][u] = 0.f;
#pragma unroll
        for (int ks = 0; ks < 4; ++ks) {
            const float* pc = s.tile + (16 * ks + 2 * c) * ld + r0 + g;
            // A = P rows r0 .., k = columns 16 ks ..: a0 (g, 2c..), a1 (g + 8, 2c..), a2 (g, 2c + 8..), a3 (g + 8, 2c + 8..)
            uint32_t ah[4], al[4];
            lf_split2(make_float2(pc[0], pc[ld]), ah[0], al[0]);
            lf_split2(make_float2(pc[8], pc[ld + 8]), ah[1], al[1]);
            lf_split2(make_float2(pc[8 * ld], pc[9 * ld]), ah[2], al[2]);
            lf_split2(make_float2(pc[8 * ld + 8], pc[9 * ld + 8]), ah[3], al[3]);
#pragma unroll
            for (int nt = 2 * ks; nt < 8; ++nt) {
                const uint4 f = s.xfrag[(ks * 8 + nt) * 32 + lane];
                lf_mma_f16(hh[nt], ah[0], ah[1], ah[2], ah[3], f.x, f.y);
                lf_mma_f16(mx[nt], ah[0], ah[1], ah[2], ah[3], f.z, f.w);
                lf_mma_f16(mx[nt], al[0], al[1], al[2], al[3], f.x, f.y);
            }
        }
        __syncwarp();   // every lane of the warp has read its rows before any of them is overwritten
#pragma unroll
        for (int nt = 0; nt < 8; ++nt) {
            const int j = 8 * nt + 2 * c;
            const float i0 = s.dsc[j], i1 = s.dsc[j + 1];
            float* o = s.tile + j * ld + r0 + g;
            o[0] = fmaf(mx[nt][0], 0x1p-11f, hh[nt][0]) * i0;
            o[ld] = fmaf(mx[nt][1], 0x1p-11f, hh[nt][1]) * i1;
            o[8] = fmaf(mx[nt][2], 0x1p-11f, hh[nt][2]) * i0;
            o[ld + 8] = fmaf(mx[nt][3], 0x1p-11f, hh[nt][3]) * i1;
        }
    }
    __syncthreads();
}

// Racc <- R_pass Racc (CTA 0, fp64, global ping-pong buffers); first pass: Racc = R_pass.
__device__ void lf_racc(const LeafArgs& a, const LfSmem& s, int pass) {
    const double* src = a.racc + (pass & 1 ? 0 : 64 * 64);
    double* dst = a.racc + (pass & 1 ? 64 * 64 : 0);
    for (int e = threadIdx.x; e < 64 * 64; e += LF_THREADS) {
        const int i = e >> 6, j = e & 63;
        double v = 0.0;
        if (i <= j) {
            if (pass == 0) {
                v = s.Rs[i * LF_GLD + j];
            } else {
                for (int k = i; k <= j; ++k) v = fma(s.Rs[i * LF_GLD + k], __ldcg(src + k * 64 + j), v);
            }
        }
        __stcg(dst + e, v);
    }
}

// Full symmetric Gram (identity beyond nc) from the packed reduced entries; optional shift.
__device__ void lf_build_g(const LfSmem& s, const double* packed, bool global, int nc, double shift) {
    for (int e = threadIdx.x; e < 64 * 64; e += LF_THREADS) {
        const int i = e >> 6, j = e & 63;
        const int lo = min(i, j), hi = max(i, j);
        const int p = hi * (hi + 1) / 2 + lo;
        double v = (i == j) ? 1.0 : 0.0;
        if (i < nc && j < nc) v = global ? __ldcg(packed + p) : packed[p];
        if (i == j && i < nc) v += shift;
        s.G[i * LF_GLD + j] = v;
        if (i == j) s.gdiag[i] = v;
    }
    __syncthreads();
}

// CholQR with the single-pass test, CholQR2 and the shifted-CholQR3 fallback.  Leaves Q in the
// tile and R in a.racc (buffer (passes - 1) & 1).  Returns the first failed pivot (or -1) and
// the number of passes through *npass.
template <int NI>
__device__ int lf_cholqr(const LeafArgs& a, const LfSmem& s, int nc, int rp, int* npass) {
    bool shifted = false;
    bool fast = a.fast != 0;   // first pass on the split-fp16 Gram (lf_gram16)
    int bad = -1;
    int pass = 0;
    for (; pass < 3; ++pass) {
        if (fast && pass == 0) lf_gram16(a, s, rp);
        else lf_gram(a, s, rp);
        if (pass == 0) LF_MARK(2);
        lf_allreduce(a, s, LF_NE, true, pass == 0 ? 20 : 0);
        if (pass == 0) LF_MARK(3);
        if (fast && pass == 0 && a.chol) {
            // the blocked fast path reads the packed Gram directly: only the diagonal is needed
            if (threadIdx.x < 64)
                s.gdiag[threadIdx.x] = threadIdx.x < nc ? s.red[threadIdx.x * (threadIdx.x + 3) / 2] : 1.0;
        } else {
            lf_build_g(s, s.red, false, nc, 0.0);
        }
        if (pass == 0) LF_MARK(26);
        if (fast && pass == 0) {
            // split-Gram validity: every column norm in [0.01, 2^15] (entries far from the fp16
            // subnormal and overflow ranges) and finite
            if (threadIdx.x == 0) s.flag[1] = 0;
            __syncthreads();
            if (threadIdx.x < nc) {
                const double d = s.gdiag[threadIdx.x];
                if (!(d >= 1e-4 && d <= 0x1p30)) s.flag[1] = 1;
            }
            __syncthreads();
            LF_MARK(27);
            if (s.flag[1]) {
                LF_COUNT(0, 1);
                fast = false;
                pass = -1;
                continue;
            }
        }
        if (fast && pass == 0) {
            // fp32 Cholesky + inverse in one loop; a failed pivot or a kappa above the fast-path
            // bound redoes the pass on the fp64 Gram
            double keq = 0.0;
            const int fb32 = a.chol ? lf_chol_inv_b4(s, nc, &keq) : lf_chol_inv32<LF_CHOL_WARPS>(s, nc, &keq);
            LF_MARK(4);
            if (fb32 < 64 || !(keq <= 1.21 * nc * nc)) {
                LF_COUNT(0, 1);
                fast = false;
                pass = -1;
                continue;
            }
            LF_MARK(5);
            lf_apply16(a, s, rp);
            LF_MARK(6);
            break;   // single pass: R in s.Rs
        }
        int fb = threadIdx.x < 128 ? lf_chol(s) : 64;
        if (threadIdx.x == 0) s.flag[0] = fb;
        __syncthreads();
        fb = s.flag[0];
        if (fb < 64 && pass == 0) {
            // shifted CholQR: G + sh I, sh = 11 (m nc + nc (nc + 1)) u ||P||_F^2
            double tr = 0.0;
            for (int i = 0; i < nc; ++i) tr += __ldcg(a.red + i * (i + 1) / 2 + i);
            const double sh = 11.0 * ((double)a.m * nc + (double)nc * (nc + 1)) * 0x1p-53 * tr;
            __syncthreads();
            lf_build_g(s, a.red, true, nc, sh);
            shifted = true;
            fb = threadIdx.x < 128 ? lf_chol(s) : 64;
            if (threadIdx.x == 0) s.flag[0] = fb;
            __syncthreads();
            fb = s.flag[0];
        }
        if (pass == 0) LF_MARK(4);
        if (fb < 64) {
            bad = fb;
            break;
        }
        const double kk = lf_inverse(s, nc);   // every thread: same value
        const bool stop = (pass == 0) ? (!shifted && kk <= 4.0 * nc * nc)
                                      : ((pass == 1 && !shifted) || pass == 2);
        // R = R_p ... R_1: a single pass keeps R in s.Rs; otherwise CTA 0 accumulates in global
        if (blockIdx.x == 0 && !(pass == 0 && stop)) lf_racc(a, s, pass);
        if (pass == 0) LF_MARK(5);
        lf_apply<NI>(a, s, rp);
        if (pass == 0) LF_MARK(6);
        if (stop) break;
    }
    *npass = pass + 1;
    LF_COUNT(1, pass + 1);
    return bad;
}

// ------------------------------------------------------------------ prologue: the level above
// R_AB = Q_A^T P (64 x 64) and P <- P - Q_A R_AB for the block's columns P (tile) and the
// preceding block's columns Q_A (16-bit image, staged in s.qa): Algorithm 1 lines 8-9 of the
// recursion level just above the leaf, in the precision of the tensor-core GEMMs (16-bit operands,
// fp32 accumulation).  Replaces that level's K1 GEMM + split-K reduce + K2 GEMM launches.
__device__ void lf_load_qa(const LeafArgs& a, const LfSmem& s, int64_t r0, int rows, int rp16) {
    const int ld16 = lf_qa_ld(rp16);
    const int nq = rp16 >> 3;   // 8-row (16-byte) chunks per column
    for (int e = threadIdx.x; e < 64 * nq; e += LF_THREADS) {
        const int cc = e / nq, q = e % nq;
        uint16_t* dst = s.qa + cc * ld16 + 8 * q;
        const uint16_t* src = a.pq + r0 + (int64_t)cc * a.ldh;
        const int avail = (cc < a.ph) ? max(0, min(8, rows - 8 * q)) : 0;
        lf_cp16(dst, avail > 0 ? src + 8 * q : src, avail * 2);
    }
}

// partial R_AB: warp w owns the 16 x 16 output block (w / 4, w % 4) over all k-steps
template <int BF>
__device__ void lf_pro_k1(const LeafArgs& a, const LfSmem& s, int rp16) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, c = lane & 3;
    const int bi = warp >> 2, bj = warp & 3;
    const int ld16 = lf_qa_ld(rp16), ld = a.ldt;
    float acc[2][4];
#pragma unroll
    for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int u = 0; u < 4; ++u) acc[nt][u] = 0.f;
    const uint16_t* qb = s.qa + (16 * bi + g) * ld16 + 2 * c;
    const float* pb = s.tile + (16 * bj + g) * ld + 2 * c;
#pragma unroll 2
    for (int k0 = 0; k0 < rp16; k0 += 16) {
        uint32_t af[4], bfr[2][2];
        af[0] = *reinterpret_cast<const uint32_t*>(qb + k0);
        af[1] = *reinterpret_cast<const uint32_t*>(qb + 8 * ld16 + k0);
        af[2] = *reinterpret_cast<const uint32_t*>(qb + k0 + 8);
        af[3] = *reinterpret_cast<const uint32_t*>(qb + 8 * ld16 + k0 + 8);
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) {
            const float2 y0 = *reinterpret_cast<const float2*>(pb + 8 * nt * ld + k0);
            const float2 y1 = *reinterpret_cast<const float2*>(pb + 8 * nt * ld + k0 + 8);
            bfr[nt][0] = lf_pack2(y0.x, y0.y, BF);
            bfr[nt][1] = lf_pack2(y1.x, y1.y, BF);
        }
#pragma unroll
        for (int nt = 0; nt < 2; ++nt) lf_mma16816(acc[nt], af, bfr[nt], BF);
    }
#pragma unroll
    for (int nt = 0; nt < 2; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int i = 16 * bi + g + 8 * h, j = 16 * bj + 8 * nt + 2 * c;   // (j, j + 1): one 16 B store
            __stcg(reinterpret_cast<double2*>(a.part + lf_pidx(i * 64 + j, blockIdx.x)),
                   make_double2((double)acc[nt][2 * h], (double)acc[nt][2 * h + 1]));
        }
}

// P <- P - Q_A R_AB over the tile's 64 columns; s.RABh holds -R_AB as [n][k]
template <int BF>
__device__ void lf_pro_k2(const LeafArgs& a, const LfSmem& s, int rp16) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, c = lane & 3;
    const int ld16 = lf_qa_ld(rp16), ld = a.ldt;
    const int kss = (a.ph + 15) >> 4;
    for (int r0 = 16 * warp; r0 < rp16; r0 += 16 * LF_NW) {
        float d[8][4];
#pragma unroll
        for (int nt = 0; nt < 8; ++nt) {
            const float* cp = s.tile + (8 * nt + 2 * c) * ld + r0 + g;
            d[nt][0] = cp[0];
            d[nt][1] = cp[ld];
            d[nt][2] = cp[8];
            d[nt][3] = cp[ld + 8];
        }
        for (int ks = 0; ks < kss; ++ks) {
            const uint16_t* q = s.qa + (16 * ks + 2 * c) * ld16 + r0 + g;
            uint32_t af[4];
            af[0] = (uint32_t)q[0] | ((uint32_t)q[ld16] << 16);
            af[1] = (uint32_t)q[8] | ((uint32_t)q[ld16 + 8] << 16);
            af[2] = (uint32_t)q[8 * ld16] | ((uint32_t)q[9 * ld16] << 16);
            af[3] = (uint32_t)q[8 * ld16 + 8] | ((uint32_t)q[9 * ld16 + 8] << 16);
#pragma unroll
            for (int nt = 0; nt < 8; ++nt) {
                const uint16_t* bp = s.RABh + (8 * nt + g) * LF_ABLD + 16 * ks + 2 * c;
                const uint32_t bfr[2] = {*reinterpret_cast<const uint32_t*>(bp),
                                         *reinterpret_cast<const uint32_t*>(bp + 8)};
                lf_mma16816(d[nt], af, bfr, BF);
            }
        }
#pragma unroll
        for (int nt = 0; nt < 8; ++nt) {
            float* cp = s.tile + (8 * nt + 2 * c) * ld + r0 + g;
            cp[0] = d[nt][0];
            cp[ld] = d[nt][1];
            cp[8] = d[nt][2];
            cp[ld + 8] = d[nt][3];
        }
    }
    __syncthreads();
}

// ------------------------------------------------------------------ load / store
__device__ void lf_load_cols(const LeafArgs& a, const LfSmem& s, int64_t r0, int rows, int rp16) {
    const int nq = rp16 >> 2;   // 4-row chunks per column
    for (int e = threadIdx.x; e < 64 * nq; e += LF_THREADS) {
        const int cc = e / nq, q = e % nq;
        float* dst = s.tile + cc * a.ldt + 4 * q;
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

template <int BF>
__device__ void lf_store_cols(const LeafArgs& a, const LfSmem& s, int64_t r0, int rows) {
    const int nq = (rows + 3) >> 2;
    for (int e = threadIdx.x; e < a.nc * nq; e += LF_THREADS) {
        const int cc = e / nq, q = e % nq;
        const float4 v = *reinterpret_cast<const float4*>(s.tile + cc * a.ldt + 4 * q);
        const int64_t gr = r0 + 4 * q;
        float* dq = a.Q + gr + (int64_t)cc * a.ldq;
        const float vv[4] = {v.x, v.y, v.z, v.w};
        ushort4 hb, lb;
        uint16_t* hbp = reinterpret_cast<uint16_t*>(&hb);
        uint16_t* lbp = reinterpret_cast<uint16_t*>(&lb);
#pragma unroll
        for (int u = 0; u < 4; ++u) hbp[u] = lf_to16(vv[u], BF);
        if (a.Ql) {   // lo image (split mode) only when requested
#pragma unroll
            for (int u = 0; u < 4; ++u) lbp[u] = lf_to16((vv[u] - lf_from16(hbp[u], BF)) * 2048.f, BF);
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

// ------------------------------------------------------------------ the kernel
template <int NI, int BF>
__global__ void __launch_bounds__(LF_THREADS, 1) leaf_kernel(LeafArgs a) {
    extern __shared__ __align__(16) uint8_t lf_smem[];
    const LfSmem s(lf_smem, a.ldt);
    const int64_t r0 = (int64_t)blockIdx.x * a.rows_per;
    const int64_t rem = a.m - r0;
    const int rows = rem <= 0 ? 0 : (rem < a.rows_per ? (int)rem : a.rows_per);
    const int rp16 = (rows + 15) & ~15;
    LF_MARK(0);
    if (blockIdx.x == 0 && threadIdx.x == 0) a.stats[0] += 1;
#ifdef LF_TRACE
    if (blockIdx.x == 0 && threadIdx.x == 0) lf_clk[0] = clock64();
#endif
    lf_load_cols(a, s, r0, rows, rp16);
    if (a.pq) lf_load_qa(a, s, r0, rows, rp16);
    lf_cp_commit();
    lf_cp_wait_all();
    __syncthreads();
    if (a.pq) {
        // ---- prologue: the level above (R_AB = Q_A^T P, P -= Q_A R_AB)
        LF_MARK(10);
        lf_pro_k1<BF>(a, s, rp16);
        LF_MARK(11);
        lf_allreduce(a, s, 4096, false);
        LF_MARK(12);
        {
            constexpr int MQ = 4096 / LF_THREADS;   // all loads in flight, then convert / store
            float v[MQ];
#pragma unroll
            for (int u = 0; u < MQ; ++u) {
                const int e = threadIdx.x + u * LF_THREADS, i = e >> 6, j = e & 63;   // R_AB(i, j)
                v[u] = (i < a.ph && j < a.nc) ? (float)__ldcg(a.red + e) : 0.f;
            }
#pragma unroll
            for (int u = 0; u < MQ; ++u) {
                const int e = threadIdx.x + u * LF_THREADS, i = e >> 6, j = e & 63;
                s.RABh[j * LF_ABLD + i] = lf_to16(-v[u], BF);
                if (blockIdx.x == 0 && i < a.ph && j < a.nc) a.R[(int64_t)(i - a.ph) + (int64_t)j * a.ldr] = v[u];
            }
        }
        __syncthreads();
        LF_MARK(13);
        lf_pro_k2<BF>(a, s, rp16);
    }
    LF_MARK(1);
    int npass = 0;
    const int bad = lf_cholqr<NI>(a, s, a.nc, rp16, &npass);
    if (bad >= 0) {   // uniform across the grid (every CTA factors the same reduced Gram)
        if (blockIdx.x == 0 && threadIdx.x == 0) atomicMin(a.status, a.col0 + bad);
        return;
    }
    LF_MARK(7);
    lf_store_cols<BF>(a, s, r0, rows);
    if (blockIdx.x == 0) {   // R (fp32) from the fp64 factor (s.Rs for one pass, else the accumulated one)
        const double* racc = a.racc + (((npass - 1) & 1) ? 64 * 64 : 0);
        for (int e = threadIdx.x; e < a.nc * a.nc; e += LF_THREADS) {
            const int i = e % a.nc, j = e / a.nc;
            const double v = npass == 1 ? s.Rs[i * LF_GLD + j] : __ldcg(racc + i * 64 + j);
            a.R[i + (int64_t)j * a.ldr] = (i <= j) ? (float)v : 0.f;
        }
    }
    LF_MARK(8);
#ifdef LF_TRACE
    if (blockIdx.x == 0 && threadIdx.x == 0) lf_clk[1] = clock64();
#endif
}

// ------------------------------------------------------------------ host side
static int lf_sms() { return dev_sms(); }
static int lf_smem_max() { return dev_smem_optin() - 1024; }   // static shared memory + slack
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

bool leaf_prologue_fits(int64_t m) {
    int grid, rows_per, ldt;
    lf_geometry(m, grid, rows_per, ldt);
    return (size_t)64 * lf_qa_ld((rows_per + 15) & ~15) * 2 <= 2 * LF_REGION;
}

size_t leaf_ws_doubles() { return (size_t)(LF_MAX_GRID + 1) * LF_PART + 2 * 64 * 64 + 64; }
size_t leaf_stats_offset() { return (size_t)(LF_MAX_GRID + 1) * LF_PART + 2 * 64 * 64; }

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
    a.racc = a.red + LF_PART;
    a.stats = reinterpret_cast<unsigned long long*>(a.racc + 2 * 64 * 64);
    a.bar = L.bar;
    a.status = L.status;
    a.col0 = L.col0;
    a.bf16 = L.bf16;
    a.pq = L.pq;
    a.ph = L.pq ? L.ph : 0;
    static const bool fp64_gram = getenv("RGSQR_LEAF_FP64_GRAM") != nullptr;
    a.fast = fp64_gram ? 0 : 1;
    static const int chol = getenv("RGSQR_LEAF_CHOL") ? atoi(getenv("RGSQR_LEAF_CHOL")) : LF_CHOL_BLOCKED;
    a.chol = chol;
    if (a.pq && (a.ph < 1 || a.ph > 64 || (L.ldh & 7) != 0 || (reinterpret_cast<uintptr_t>(L.pq) & 15) != 0 ||
                 !leaf_prologue_fits(L.m)))
        return cudaErrorInvalidValue;
    int grid;
    lf_geometry(L.m, grid, a.rows_per, a.ldt);
    a.vec = ((L.ldq & 3) == 0) && ((reinterpret_cast<uintptr_t>(L.Q) & 15) == 0) && ((L.ldh & 3) == 0) &&
            ((reinterpret_cast<uintptr_t>(L.Qh) & 7) == 0) && ((reinterpret_cast<uintptr_t>(L.Ql) & 7) == 0);
    const size_t smem = leaf_smem_bytes(L.m);
    const bool small = ((a.rows_per + 15) & ~15) <= 448;
    // the 16-bit format is a template parameter: runtime bf16 branches in the prologue's mma.sync /
    // pack loops and the image stores cost convergence-barrier (BSSY) overhead
    void (*kern)(LeafArgs) = a.bf16 ? (small ? leaf_kernel<7, 1> : leaf_kernel<LF_MAXI, 1>)
                                    : (small ? leaf_kernel<7, 0> : leaf_kernel<LF_MAXI, 0>);
    {
        cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(kern), smem);
        if (e != cudaSuccess) return e;
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
