// tall.cu -- one CholQR pass over a whole tall-skinny block (n <= 256 columns, m >> n) on the
// tcgen05 tensor cores, the base case of Algorithm 1 for `orthogonalize`
// (config 4) when the block is too tall for the on-chip leaf (reading #33):
//
//   G = X^T X                     tl_gram_kernel: two-term 16-bit split of every entry, three
//                                 tcgen05 products into one fp32 TMEM accumulator per CTA;
//                                 the diagonal (column norms) summed exactly in fp64 beside it
//   G -> fp64, fixed order        tl_reduce_kernel (+ NCCL / virtual-rank allreduce when row-sharded)
//   G = D G^ D, G^ = R^T R^       tl_chol_kernel: fp64 equilibration, fp32 Cholesky and R^-1 of the
//                                 unit-diagonal G^ (one CTA); R = R^ D, breakdown / kappa check
//   X <- X R^-1                   tl_apply_kernel: in place, X D^-1 split on the fly, R^^-1 split
//                                 and resident in shared memory (upper triangle only), three
//                                 tcgen05 products per k-block into a TMEM accumulator
//
// The 16-bit split (reading #9, reading #33): x = hi + lo with hi = rn16(s x), lo = rn16(s x - hi)
// (unscaled lo, so all three products accumulate into ONE accumulator; the per-column or per-pass
// power-of-two scale s keeps lo in the normal 16-bit range).  The first pass's Gram in bf16 (fp32
// exponent range: no column scaling pass needed before it), every other Gram and every apply in
// fp16 (22-bit split) at 2^14 on unit columns (the apply scales X by D^-1 from the Gram).
//
// fp32 X is read straight from HBM by 8 converter warps (16-byte loads, 64 rows of a column per
// half-warp) that write the swizzled 128-byte lines of the UMMA operands (SWIZZLE_128B: K-major
// lines for the Gram, MN-major lines for the apply -- the same physical layout: one line = 64
// consecutive rows of one column).  One CTA per SM, persistent over row chunks.
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>

#include <cmath>
#include <cstdlib>

#include "kernels.h"
#include "ptx.cuh"

namespace rg {

constexpr int TL_N = 256;                    // padded columns
constexpr int TL_CW = 8;                     // converter warps (warps 4..11)
constexpr int TL_THREADS = 128 + 32 * TL_CW;
constexpr int TL_GSTAGES = 3;
constexpr int TL_GSTAGE = 2 * TL_N * 128;    // hi + lo tiles of one Gram stage (64 rows x 256 cols)
constexpr int TL_GACC = 384;                 // TMEM columns: D0 (128 x 256) + D1 (128 x 128)
constexpr int TL_PART = TL_GACC * 128;       // fp32 per CTA partial (three-product Gram: D0 | D1)
constexpr int TL_PART2 = 512 * 128;          // two-product Gram: full 256 x 256 D = H (H + 2L)^T
constexpr int TL_PMAX = TL_PART2;
constexpr int TL_ASTAGES = 2;
constexpr int TL_ASTAGE = 2 * 64 * 256;      // hi + lo of one apply k-block (128 rows x 64 cols)
constexpr int TL_BBYTES = (256 + 192 + 128 + 64) * 128;   // one of hi / lo of the resident R^-1 tiles
constexpr int TL_MAX_GRID = 160;

__device__ __forceinline__ uint32_t tl_pack(float a, float b, bool bf) {
    if (bf) {
        __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
        return *reinterpret_cast<uint32_t*>(&v);
    }
    __half2 v = __floats2half2_rn(a, b);
    return *reinterpret_cast<uint32_t*>(&v);
}
__device__ __forceinline__ float2 tl_unpack(uint32_t u, bool bf) {
    if (bf) return __bfloat1622float2(*reinterpret_cast<__nv_bfloat162*>(&u));
    return __half22float2(*reinterpret_cast<__half2*>(&u));
}

__device__ __forceinline__ void tl_sts64(uint32_t addr, uint32_t a, uint32_t b) {
    asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(addr), "r"(a), "r"(b) : "memory");
}
__device__ __forceinline__ float4 tl_lds128(uint32_t addr) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(addr));
    return v;
}
// 4 consecutive rows (one float4, already scaled) -> 8 bytes of hi at shared address hi_addr and
// of lo at lo_addr (swizzled by the caller)
// (LS: lo scale, 1 or 2 -- a power of two, so rn16(LS (x - hi)) = LS rn16(x - hi) exactly)
template <bool BF, int LS = 1>
__device__ __forceinline__ void tl_split_sts(float4 v, uint32_t hi_addr, uint32_t lo_addr) {
    const uint32_t h0 = tl_pack(v.x, v.y, BF), h1 = tl_pack(v.z, v.w, BF);
    const float2 a = tl_unpack(h0, BF), b = tl_unpack(h1, BF);
    const float ls = (float)LS;
    const uint32_t l0 = tl_pack(ls * (v.x - a.x), ls * (v.y - a.y), BF), l1 = tl_pack(ls * (v.z - b.x), ls * (v.w - b.y), BF);
    tl_sts64(hi_addr, h0, h1);
    tl_sts64(lo_addr, l0, l1);
}

// SWIZZLE_128B byte offset of the 8-byte piece g (0..15) of line `line` (1024-byte aligned tile)
__device__ __forceinline__ uint32_t tl_swz(int line, int g) {
    return (uint32_t)line * 128u + ((uint32_t)(((g >> 1) ^ (line & 7)) << 4)) + (uint32_t)((g & 1) << 3);
}

// rows [r, r + 4) of one column (16-byte aligned when vec), zero beyond m
__device__ __forceinline__ float4 tl_load4(const float* col, int64_t r, int64_t m, bool vec) {
    if (vec && r + 4 <= m) return __ldcs(reinterpret_cast<const float4*>(col + r));
    float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
    if (r < m) v.x = col[r];
    if (r + 1 < m) v.y = col[r + 1];
    if (r + 2 < m) v.z = col[r + 2];
    if (r + 3 < m) v.w = col[r + 3];
    return v;
}

// ======================================================================= Gram
struct TlGramArgs {
    const float* X;
    int64_t ldx;
    int64_t m;
    int n;
    float sig;          // conversion scale (power of two)
    int vec;            // 16-byte loads allowed
    float* part;        // [grid][TL_PART]
    double* npart;      // [grid][TL_N] column sums of (sig x)^2
};

template <bool BF>
__global__ void __launch_bounds__(TL_THREADS, 1) tl_gram_kernel(TlGramArgs a) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint64_t* full_bar = reinterpret_cast<uint64_t*>(smem + TL_GSTAGES * TL_GSTAGE);
    uint64_t* empty_bar = full_bar + TL_GSTAGES;
    uint64_t* done_bar = empty_bar + TL_GSTAGES;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(done_bar + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t nchunks = (a.m + 63) / 64;
    const int my = nchunks > blockIdx.x ? (int)((nchunks - 1 - blockIdx.x) / gridDim.x + 1) : 0;

    if (threadIdx.x == 0) {
        for (int s = 0; s < TL_GSTAGES; ++s) {
            mbar_init(&full_bar[s], TL_CW);
            mbar_init(&empty_bar[s], 1);
        }
        mbar_init(done_bar, 1);
        fence_barrier_init();
    }
    if (warp == 1) tmem_alloc<512>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    RG_PDL_ENTRY();

    if (warp == 0) {
        if (elect_one()) {
            // ---------------- MMA issuer: D0 = G[0:128, 0:256], D1 = G[128:256, 128:256]
            const uint32_t id256 = umma_idesc_f16(128, 256, 0, 0, BF ? 1u : 0u);
            const uint32_t id128 = umma_idesc_f16(128, 128, 0, 0, BF ? 1u : 0u);
            for (int it = 0; it < my; ++it) {
                const int s = it % TL_GSTAGES;
                mbar_wait(&full_bar[s], (uint32_t)(it / TL_GSTAGES) & 1u);
                tc_fence_after();
                const uint32_t hi = smem_u32(smem + s * TL_GSTAGE);
                const uint32_t lo = hi + TL_N * 128;
#pragma unroll
                for (int kk = 0; kk < 4; ++kk) {
                    const uint32_t acc = (it > 0 || kk > 0) ? 1u : 0u;
                    const uint64_t h0 = umma_desc_sw128(hi + kk * 32, 16, 1024);
                    const uint64_t l0 = umma_desc_sw128(lo + kk * 32, 16, 1024);
                    const uint64_t h1 = umma_desc_sw128(hi + 128 * 128 + kk * 32, 16, 1024);
                    const uint64_t l1 = umma_desc_sw128(lo + 128 * 128 + kk * 32, 16, 1024);
                    umma_f16(tmem, h0, h0, id256, acc);
                    umma_f16(tmem, h0, l0, id256, 1u);
                    umma_f16(tmem, l0, h0, id256, 1u);
                    umma_f16(tmem + 256, h1, h1, id128, acc);
                    umma_f16(tmem + 256, h1, l1, id128, 1u);
                    umma_f16(tmem + 256, l1, h1, id128, 1u);
                }
                umma_commit(&empty_bar[s]);
            }
            umma_commit(done_bar);
        }
        __syncwarp();
    } else if (warp >= 4) {
        // ---------------- converters: column pair cp = 16 cw + p, column 2 cp + (lane >> 4),
        // rows 4 (lane & 15) .. + 3 of the 64-row chunk
        const int cw = warp - 4;
        const int g = lane & 15;
        double nrm[16];
        float nf[16];
#pragma unroll
        for (int p = 0; p < 16; ++p) {
            nrm[p] = 0.0;
            nf[p] = 0.f;
        }
        for (int it = 0; it < my; ++it) {
            const int s = it % TL_GSTAGES;
            const int64_t r0 = ((int64_t)blockIdx.x + (int64_t)it * gridDim.x) * 64 + 4 * g;
            float4 v[16];
#pragma unroll
            for (int p = 0; p < 16; ++p) {
                const int c = 2 * (16 * cw + p) + (lane >> 4);
                v[p] = c < a.n ? tl_load4(a.X + (int64_t)c * a.ldx, r0, a.m, a.vec != 0) : make_float4(0.f, 0.f, 0.f, 0.f);
            }
            mbar_wait(&empty_bar[s], ((uint32_t)(it / TL_GSTAGES) & 1u) ^ 1u);
            uint8_t* hi = smem + s * TL_GSTAGE;
            uint8_t* lo = hi + TL_N * 128;
#pragma unroll
            for (int p = 0; p < 16; ++p) {
                const int c = 2 * (16 * cw + p) + (lane >> 4);
                float4 x = v[p];
                nf[p] = fmaf(x.x, x.x, fmaf(x.y, x.y, fmaf(x.z, x.z, fmaf(x.w, x.w, nf[p]))));
                x.x *= a.sig; x.y *= a.sig; x.z *= a.sig; x.w *= a.sig;
                const uint32_t off = tl_swz(c, g);
                tl_split_sts<BF>(x, smem_u32(hi) + off, smem_u32(lo) + off);
            }
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(&full_bar[s]);
            if ((it & 31) == 31) {
#pragma unroll
                for (int p = 0; p < 16; ++p) {
                    nrm[p] += (double)nf[p];
                    nf[p] = 0.f;
                }
            }
        }
        // column norms: 16 lanes share a column
#pragma unroll
        for (int p = 0; p < 16; ++p) {
            double x = nrm[p] + (double)nf[p];
#pragma unroll
            for (int o = 1; o < 16; o <<= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
            if (g == 0) a.npart[(int64_t)blockIdx.x * TL_N + 2 * (16 * cw + p) + (lane >> 4)] = x * (double)a.sig * (double)a.sig;
        }
        // ---------------- epilogue: TMEM -> partial [col][lane]
        const int q = warp & 3, half = cw >> 2;
        float* P = a.part + (int64_t)blockIdx.x * TL_PART;
        if (my > 0) {
            mbar_wait(done_bar, 0);
            tc_fence_after();
        }
        for (int ch = half; ch < TL_GACC / 32; ch += 2) {
            uint32_t r[32];
            if (my > 0) {
                tmem_ld32(tmem + ((uint32_t)(32 * q) << 16) + ch * 32, r);
                tmem_ld_wait();
            } else {
#pragma unroll
                for (int j = 0; j < 32; ++j) r[j] = 0u;
            }
#pragma unroll
            for (int j = 0; j < 32; ++j) P[(int64_t)(ch * 32 + j) * 128 + 32 * q + lane] = __uint_as_float(r[j]);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1) tmem_dealloc<512>(tmem);
}

// TMA-fed variant (16-byte aligned X and ldx): a producer warp streams 64-row x 128-column fp32
// half-chunks of X (256 contiguous bytes per column: 32-row boxes cap HBM reads at ~4.7 TB/s,
// tools/colread_probe.cu) into a ring of three 32 KB staging slots, 16 converter warps split them
// from shared memory into the two operand stages.  Two split products, D = H (H + 2L)^T over the
// full 256 x 256 (512 TMEM columns); G = (D + D^T) / 2 = H H^T + H L^T + L H^T after the reduction.
constexpr int TL_TSLOTS = 3;
constexpr int TL_TSLOT = 32 * TL_N * 4;
constexpr int TL_TSTAGES = 2;
constexpr int TL_TCW = 16;                     // converter warps of the TMA-fed Gram
constexpr int TL_TTHREADS = 128 + 32 * TL_TCW;
constexpr int TL_GRAM_TMA_SMEM = TL_TSTAGES * TL_GSTAGE + TL_TSLOTS * TL_TSLOT + 256 + 1024;

template <bool BF>
__global__ void __launch_bounds__(TL_TTHREADS, 1) tl_gram_tma_kernel(const __grid_constant__ CUtensorMap tmX,
                                                                    TlGramArgs a) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t* stg = smem + TL_TSTAGES * TL_GSTAGE;
    uint64_t* full_bar = reinterpret_cast<uint64_t*>(stg + TL_TSLOTS * TL_TSLOT);
    uint64_t* empty_bar = full_bar + TL_TSTAGES;
    uint64_t* sfull = empty_bar + TL_TSTAGES;
    uint64_t* sempty = sfull + TL_TSLOTS;
    uint64_t* done_bar = sempty + TL_TSLOTS;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(done_bar + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t nchunks = (a.m + 63) / 64;
    const int my = nchunks > blockIdx.x ? (int)((nchunks - 1 - blockIdx.x) / gridDim.x + 1) : 0;

    if (threadIdx.x == 0) {
        tma_prefetch_desc(&tmX);
        for (int s = 0; s < TL_TSTAGES; ++s) {
            mbar_init(&full_bar[s], TL_TCW);
            mbar_init(&empty_bar[s], 1);
        }
        for (int s = 0; s < TL_TSLOTS; ++s) {
            mbar_init(&sfull[s], 1);
            mbar_init(&sempty[s], TL_TCW);
        }
        mbar_init(done_bar, 1);
        fence_barrier_init();
    }
    if (warp == 1) tmem_alloc<512>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    RG_PDL_ENTRY();

    if (warp == 0) {
        if (elect_one()) {
            // D0 = rows 0..127, D1 = rows 128..255 of D = H H^T + H (2L)^T (all 256 columns; the
            // symmetric part of D is G, formed after the reduction)
            const uint32_t id256 = umma_idesc_f16(128, 256, 0, 0, BF ? 1u : 0u);
            for (int it = 0; it < my; ++it) {
                const int s = it % TL_TSTAGES;
                mbar_wait(&full_bar[s], (uint32_t)(it / TL_TSTAGES) & 1u);
                tc_fence_after();
                const uint32_t hi = smem_u32(smem + s * TL_GSTAGE);
                const uint32_t lo = hi + TL_N * 128;
#pragma unroll
                for (int kk = 0; kk < 4; ++kk) {
                    const uint32_t acc = (it > 0 || kk > 0) ? 1u : 0u;
                    const uint64_t h0 = umma_desc_sw128(hi + kk * 32, 16, 1024);
                    const uint64_t l0 = umma_desc_sw128(lo + kk * 32, 16, 1024);
                    const uint64_t h1 = umma_desc_sw128(hi + 128 * 128 + kk * 32, 16, 1024);
                    umma_f16(tmem, h0, h0, id256, acc);
                    umma_f16(tmem, h0, l0, id256, 1u);
                    umma_f16(tmem + 256, h1, h0, id256, acc);
                    umma_f16(tmem + 256, h1, l0, id256, 1u);
                }
                umma_commit(&empty_bar[s]);
            }
            umma_commit(done_bar);
        }
        __syncwarp();
    } else if (warp == 2) {
        if (elect_one()) {
            // ---------------- TMA producer: half-chunk q = rows [64 (cta + grid (q >> 1)) + 32 (q & 1), +32)
            for (int q = 0; q < 2 * my; ++q) {
                const int sl = q % TL_TSLOTS;
                mbar_wait(&sempty[sl], ((uint32_t)(q / TL_TSLOTS) & 1u) ^ 1u);
                mbar_arrive_expect_tx(&sfull[sl], TL_TSLOT);
                const int64_t r0 = ((int64_t)blockIdx.x + (int64_t)(q >> 1) * gridDim.x) * 64;
                tma_load_2d(stg + sl * TL_TSLOT, &tmX, &sfull[sl], (int32_t)r0, 128 * (q & 1));
            }
        }
        __syncwarp();
    } else if (warp >= 4) {
        // ---------------- converters: half-chunk q = 64 rows x 128 columns (128 hf + c), staging layout
        // [column][64 rows] (256 contiguous bytes per column: 64-row segments stream at ~6.4 TB/s,
        // 32-row ones at ~4.7, tools/colread_probe.cu); a half-warp takes one column (4 rows per
        // lane), warp cw the column pairs 2 (4 cw + k) + (lane >> 4), k < 4: full 128-byte lines
        const int cw = warp - 4, g = lane & 15, hsel = lane >> 4;
        double nrm[8];
        float nf[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            nrm[k] = 0.0;
            nf[k] = 0.f;
        }
        for (int q = 0; q < 2 * my; ++q) {
            const int sl = q % TL_TSLOTS, it = q >> 1, hf = q & 1, s = it % TL_TSTAGES;
            mbar_wait(&sfull[sl], (uint32_t)(q / TL_TSLOTS) & 1u);
            if (hf == 0) mbar_wait(&empty_bar[s], ((uint32_t)(it / TL_TSTAGES) & 1u) ^ 1u);
            const uint32_t src = smem_u32(stg + sl * TL_TSLOT);
            uint8_t* hi = smem + s * TL_GSTAGE;
            uint8_t* lo = hi + TL_N * 128;
            float4 v[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const int cl = 2 * (4 * cw + k) + hsel;   // column within the half
                v[k] = tl_lds128(src + (uint32_t)(cl * 256 + 16 * g));
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&sempty[sl]);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const int c = 128 * hf + 2 * (4 * cw + k) + hsel;
                float4 x = v[k];
                nf[4 * hf + k] = fmaf(x.x, x.x, fmaf(x.y, x.y, fmaf(x.z, x.z, fmaf(x.w, x.w, nf[4 * hf + k]))));
                x.x *= a.sig; x.y *= a.sig; x.z *= a.sig; x.w *= a.sig;
                const uint32_t off = tl_swz(c, g);
                tl_split_sts<BF, 2>(x, smem_u32(hi) + off, smem_u32(lo) + off);
            }
            if (hf == 1) {
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) mbar_arrive(&full_bar[s]);
            }
            if ((q & 31) == 31) {   // fp32 partial sums of <= 64 squares, then fp64
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    nrm[k] += (double)nf[k];
                    nf[k] = 0.f;
                }
            }
        }
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            double x = nrm[k] + (double)nf[k];
#pragma unroll
            for (int o = 1; o < 16; o <<= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
            const int c = 128 * (k >> 2) + 2 * (4 * cw + (k & 3)) + hsel;
            if (g == 0) a.npart[(int64_t)blockIdx.x * TL_N + c] = x * (double)a.sig * (double)a.sig;
        }
        const int qd = warp & 3, part = cw >> 2;
        float* P = a.part + (int64_t)blockIdx.x * TL_PART2;
        if (my > 0) {
            mbar_wait(done_bar, 0);
            tc_fence_after();
        }
        for (int ch = part; ch < 512 / 32; ch += TL_TCW / 4) {
            uint32_t r[32];
            if (my > 0) {
                tmem_ld32(tmem + ((uint32_t)(32 * qd) << 16) + ch * 32, r);
                tmem_ld_wait();
            } else {
#pragma unroll
                for (int j = 0; j < 32; ++j) r[j] = 0u;
            }
#pragma unroll
            for (int j = 0; j < 32; ++j) P[(int64_t)(ch * 32 + j) * 128 + 32 * qd + lane] = __uint_as_float(r[j]);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1) tmem_dealloc<512>(tmem);
}

// G (fp64, n x n, column-major ld n): strict upper triangle from the TMEM partials, diagonal from
// the fp64 column sums, lower triangle zero; every entry summed over the CTAs in a fixed order.
__global__ void __launch_bounds__(256) tl_reduce_kernel(const float* __restrict__ part, const double* __restrict__ npart,
                                                         int nb, int n, double* G, double* dbg) {
    RG_PDL_ENTRY();
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e < TL_PART) {
        const int jp = e >> 7, i = e & 127;
        const int row = jp < 256 ? i : 128 + i;
        const int col = jp < 256 ? jp : 128 + (jp - 256);
        if (col >= n) return;
        double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
        int b = 0;
        for (; b + 4 <= nb; b += 4) {
            s0 += (double)part[(int64_t)b * TL_PART + e];
            s1 += (double)part[(int64_t)(b + 1) * TL_PART + e];
            s2 += (double)part[(int64_t)(b + 2) * TL_PART + e];
            s3 += (double)part[(int64_t)(b + 3) * TL_PART + e];
        }
        for (; b < nb; ++b) s0 += (double)part[(int64_t)b * TL_PART + e];
        const double s = (s0 + s1) + (s2 + s3);
        if (row < col) {
            G[row + (int64_t)col * n] = s;
            G[col + (int64_t)row * n] = 0.0;
        } else if (row == col && dbg) {
            dbg[row] = s;   // the tensor-core diagonal (diagnostics: RGSQR_TALL_DEBUG)
        }
    } else if (e < TL_PART + TL_N) {
        const int c = e - TL_PART;
        if (c >= n) return;
        double s = 0.0;
        for (int b = 0; b < nb; ++b) s += npart[(int64_t)b * TL_N + c];
        G[c + (int64_t)c * n] = s;
    }
}

// Two-product layout: D (fp64 sum over the CTAs, fixed order) into G (n x n, both triangles),
// diagonal from the fp64 column sums; then tl_sym_kernel sets G_ij = G_ji = (D_ij + D_ji) / 2.
__global__ void __launch_bounds__(256) tl_reduce2_kernel(const float* __restrict__ part, const double* __restrict__ npart,
                                                          int nb, int n, double* G) {
    RG_PDL_ENTRY();
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e < TL_PART2) {
        const int jp = e >> 7, i = e & 127;
        const int row = jp < 256 ? i : 128 + i;
        const int col = jp & 255;
        if (row >= n || col >= n || row == col) return;
        double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
        int b = 0;
        for (; b + 4 <= nb; b += 4) {
            s0 += (double)part[(int64_t)b * TL_PART2 + e];
            s1 += (double)part[(int64_t)(b + 1) * TL_PART2 + e];
            s2 += (double)part[(int64_t)(b + 2) * TL_PART2 + e];
            s3 += (double)part[(int64_t)(b + 3) * TL_PART2 + e];
        }
        for (; b < nb; ++b) s0 += (double)part[(int64_t)b * TL_PART2 + e];
        G[row + (int64_t)col * n] = (s0 + s1) + (s2 + s3);
    } else if (e < TL_PART2 + TL_N) {
        const int c = e - TL_PART2;
        if (c >= n) return;
        double s = 0.0;
        for (int b = 0; b < nb; ++b) s += npart[(int64_t)b * TL_N + c];
        G[c + (int64_t)c * n] = s;
    }
}
// 32 x 32 tile pairs (upper tile (I, J) with its transpose (J, I)) through shared memory
__global__ void __launch_bounds__(1024) tl_sym_kernel(double* G, int n) {
    RG_PDL_ENTRY();
    __shared__ double tu[32][33], tl[32][33];
    const int I = blockIdx.x, J = blockIdx.y;
    if (I > J) return;
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const int r = 32 * I + tx, c = 32 * J + ty;          // upper tile element (r, c)
    const int r2 = 32 * J + tx, c2 = 32 * I + ty;        // lower tile element (r2, c2)
    tu[ty][tx] = (r < n && c < n) ? G[r + (int64_t)c * n] : 0.0;
    tl[ty][tx] = (r2 < n && c2 < n) ? G[r2 + (int64_t)c2 * n] : 0.0;
    __syncthreads();
    // upper (r, c) with lower (c, r): lower (c, r) = tl at (row c = 32 J + ty, col r = 32 I + tx)
    if (r < n && c < n && r != c) {
        const double v = 0.5 * (tu[ty][tx] + tl[tx][ty]);
        G[r + (int64_t)c * n] = v;
        G[c + (int64_t)r * n] = v;
    }
}

// ======================================================================= Cholesky + inverse
struct TlCholArgs {
    const double* G;    // n x n, ld n (upper triangle + diagonal)
    int n;
    double sig_g;       // the Gram's conversion scale
    float sig_a;        // the apply's conversion scale (power of two)
    int fp16;           // apply in fp16: scale R^^-1 by a power of two into the fp16 range
    double kappa_max;   // accept when kappa_F(R^) <= kappa_max
    float* R;           // n x n, ldr: R = R^ D (memory units), lower triangle zeroed
    int64_t ldr;
    float* rinv;        // [TL_N x TL_N] column-major, R^^-1 (scaled by rho), zero-padded
    float* cscale;      // [TL_N] apply column scale sig_a / d_k (0 beyond n)
    float* escale;      // [1] apply output scale 1 / (sig_a rho)
    int* flag;          // set to 1 on a breakdown / kappa test failure (the apply then does nothing)
    double* kout;       // [2] kappa_F(R^) estimate, first failed pivot (diagnostics)
};

// Blocked on 32 x 32 tiles (8 x 8 tile grid, upper triangle: 36 tiles, row-major, row stride 36
// floats so that rows are 16-byte aligned).  Tile products C op= A^T B ("TN") or A B ("NN") with a
// 4 x 4 register tile per thread, 64 threads per output tile (8 tiles in flight on 512 threads).
constexpr int TC_LD = 36;
constexpr int TC_TILE = 32 * TC_LD;
constexpr int TC_NT = 8;
__device__ __forceinline__ int tc_idx(int ib, int jb) { return jb * (jb + 1) / 2 + ib; }   // ib <= jb

template <bool TA>
__device__ __forceinline__ void tc_prod(const float* __restrict__ A, const float* __restrict__ B, int l0, int l1,
                                        int ti, int tj, float (&c)[4][4]) {
    for (int l = l0; l < l1; ++l) {
        float a[4];
        if (TA) {
            const float4 v = *reinterpret_cast<const float4*>(A + l * TC_LD + 4 * ti);
            a[0] = v.x; a[1] = v.y; a[2] = v.z; a[3] = v.w;
        } else {
#pragma unroll
            for (int r = 0; r < 4; ++r) a[r] = A[(4 * ti + r) * TC_LD + l];
        }
        const float4 b = *reinterpret_cast<const float4*>(B + l * TC_LD + 4 * tj);
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            c[r][0] = fmaf(a[r], b.x, c[r][0]);
            c[r][1] = fmaf(a[r], b.y, c[r][1]);
            c[r][2] = fmaf(a[r], b.z, c[r][2]);
            c[r][3] = fmaf(a[r], b.w, c[r][3]);
        }
    }
}
__device__ __forceinline__ void tc_zero(float (&c)[4][4]) {
#pragma unroll
    for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int s = 0; s < 4; ++s) c[r][s] = 0.f;
}
__device__ __forceinline__ void tc_store(float* C, int ti, int tj, const float (&c)[4][4], float alpha) {
#pragma unroll
    for (int r = 0; r < 4; ++r)
        *reinterpret_cast<float4*>(C + (4 * ti + r) * TC_LD + 4 * tj) =
            make_float4(alpha * c[r][0], alpha * c[r][1], alpha * c[r][2], alpha * c[r][3]);
}

// One warp: Cholesky of the 32 x 32 diagonal tile T (upper part, row-major, stride TC_LD), R into T,
// its inverse into X.  Lane j keeps column j in registers; the pivot row travels through shared
// memory (no shuffles: inside a one-warp branch the compiler's collective shuffle sequence costs
// ~300 cycles per pivot, tools/wchol_probe.cu):
//   step k: p = T(k, k), r(k, j) = c_k / sqrt(p); every lane reads row k (T(k, i), i > k: the
//   values lane i published at step k - 1) and updates c_i -= r(k, i) r(k, j); lane j then
//   publishes its new c_{k+1} as T(k + 1, j).
// X = R^-1 column-parallel (lane j: column j), right-looking: x_k /= r_kk, x_i -= r_ik x_k (i < k).
// Returns false (uniform) on a non-positive pivot.
__device__ __forceinline__ bool tc_diag(float* T, float* X, int lane) {
    float c[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) c[i] = T[i * TC_LD + lane];
    bool ok = true;
    __syncwarp();
#pragma unroll
    for (int k = 0; k < 32; ++k) {
        const float p = T[k * TC_LD + k];
        ok = ok && (p > 1e-30f);
        const float rs = __frsqrt_rn(fmaxf(p, 1e-30f));
        const float rk = c[k] * rs;   // r(k, lane), lane >= k
        c[k] = rk;
#pragma unroll
        for (int i = k + 1; i < 32; ++i) c[i] = fmaf(-(T[k * TC_LD + i] * rs), rk, c[i]);
        __syncwarp();
        if (k < 31) T[(k + 1) * TC_LD + lane] = c[k + 1];
        __syncwarp();
    }
#pragma unroll
    for (int i = 0; i < 32; ++i) T[i * TC_LD + lane] = i <= lane ? c[i] : 0.f;
    __syncwarp();
    float x[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) x[i] = i == lane ? 1.f : 0.f;
#pragma unroll
    for (int k = 31; k >= 0; --k) {
        x[k] = x[k] * __frcp_rn(T[k * TC_LD + k]);
#pragma unroll
        for (int i = 0; i < k; ++i) x[i] = fmaf(-T[i * TC_LD + k], x[k], x[i]);
    }
#pragma unroll
    for (int i = 0; i < 32; ++i) X[i * TC_LD + lane] = x[i];
    return __all_sync(0xffffffffu, ok);
}

constexpr int TC_THREADS = 512;   // 128 registers per thread: the warp-register diagonal code does not spill
constexpr int TC_NW = TC_THREADS / 32;
constexpr int TC_TASKS = TC_THREADS / 64;
__global__ void __launch_bounds__(TC_THREADS, 1) tl_chol_kernel(TlCholArgs a) {
    extern __shared__ __align__(16) float tsm[];
    float* Tl = tsm;                               // 36 tiles of the upper triangle
    float* XD = Tl + 36 * TC_TILE;                 // 8 inverted diagonal tiles
    float* TMP = XD;                               // scratch tiles of the inverse (XD is moved out first)
    double* d = reinterpret_cast<double*>(XD + TC_NT * TC_TILE);   // [TL_N]
    __shared__ int bad;
    __shared__ float gmax;
    __shared__ double red[3][TC_NW];
    RG_PDL_ENTRY();
    const int n = a.n, t = threadIdx.x, warp = t >> 5, lane = t & 31;
    const int nt = (n + 31) / 32;
    if (t == 0) {
        bad = 0;
        gmax = 0.f;
    }
    for (int i = t; i < TL_N; i += blockDim.x) {
        if (i < n) {
            const double g = a.G[i + (int64_t)i * n];
            d[i] = sqrt(g);
            if (!(g > 0.0) || !isfinite(g)) atomicMax(&bad, 1);
        } else {
            d[i] = 1.0;
        }
    }
    __syncthreads();
    if (bad) {
        if (t == 0) *a.flag = 1;
        return;
    }
    // equilibrated G^ = D^-1 G D^-1 (unit diagonal) in fp32 tiles; identity beyond n
    double* dinv = d + TL_N;
    for (int i = t; i < TL_N; i += blockDim.x) dinv[i] = 1.0 / d[i];
    __syncthreads();
    float lmax = 0.f;
    for (int j = warp; j < nt * 32; j += TC_NW)
        for (int i = lane; i <= j; i += 32) {
            const int ib = i >> 5, jb = j >> 5;
            if (ib > jb) continue;
            float v;
            if (i == j) v = 1.0f;
            else if (i > j || j >= n) v = 0.f;
            else {
                v = (float)(a.G[i + (int64_t)j * n] * dinv[i] * dinv[j]);
                lmax = fmaxf(lmax, fabsf(v));
            }
            Tl[tc_idx(ib, jb) * TC_TILE + (i & 31) * TC_LD + (j & 31)] = v;
        }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) lmax = fmaxf(lmax, __shfl_xor_sync(0xffffffffu, lmax, o));
    if (lane == 0) atomicMax(reinterpret_cast<int*>(&gmax), __float_as_int(lmax));
    __syncthreads();
    const int task = t >> 6, tl = t & 63;
    const int ti = ((tl & 31) >> 3) + 4 * (tl >> 5), tj = tl & 7;
    if (gmax <= 4e-6f) {
        // first order (reorthogonalisation passes): with |g_ij| <= eps, R^ = I + triu(G^ - I) and
        // R^^-1 = I - triu(G^ - I) up to n eps^2 <= 4e-9, below fp32 rounding; XD = R^-1 tiles, the
        // upper tiles keep R^ until the output loop below
        for (int e = t; e < nt * 32 * 32; e += blockDim.x) {
            const int kb = e >> 10, i = (e >> 5) & 31, j = e & 31;
            const float v = Tl[tc_idx(kb, kb) * TC_TILE + i * TC_LD + j];
            XD[kb * TC_TILE + i * TC_LD + j] = i == j ? 1.0f : (i < j ? -v : 0.f);
        }
        __syncthreads();
    } else {
        // right-looking blocked Cholesky
        for (int kb = 0; kb < nt; ++kb) {
            if (warp == 0) {
                const bool ok = tc_diag(Tl + tc_idx(kb, kb) * TC_TILE, XD + kb * TC_TILE, lane);
                if (!ok && lane == 0) {
                    bad = 1;
                    a.kout[1] = 32.0 * kb;
                }
            }
            __syncthreads();
            if (bad) break;
            // panel: R(kb, jb) = X_kk^T S(kb, jb)
            float c[4][4];
            const int np = nt - kb - 1;
            if (task < np) {
                tc_zero(c);
                tc_prod<true>(XD + kb * TC_TILE, Tl + tc_idx(kb, kb + 1 + task) * TC_TILE, 0, 32, ti, tj, c);
            }
            __syncthreads();
            if (task < np) tc_store(Tl + tc_idx(kb, kb + 1 + task) * TC_TILE, ti, tj, c, 1.0f);
            __syncthreads();
            // trailing: S(ib, jb) -= R(kb, ib)^T R(kb, jb), kb < ib <= jb
            const int ntr = np * (np + 1) / 2;
            for (int q = task; q < ntr; q += TC_TASKS) {
                int jj = 0;
                while ((jj + 1) * (jj + 2) / 2 <= q) ++jj;
                const int ii = q - jj * (jj + 1) / 2;
                const int ib = kb + 1 + ii, jb = kb + 1 + jj;
                float* C = Tl + tc_idx(ib, jb) * TC_TILE;
                tc_zero(c);
                tc_prod<true>(Tl + tc_idx(kb, ib) * TC_TILE, Tl + tc_idx(kb, jb) * TC_TILE, 0, 32, ti, tj, c);
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    float4* p = reinterpret_cast<float4*>(C + (4 * ti + r) * TC_LD + 4 * tj);
                    float4 v = *p;
                    v.x -= c[r][0]; v.y -= c[r][1]; v.z -= c[r][2]; v.w -= c[r][3];
                    *p = v;
                }
            }
            __syncthreads();
        }
        if (bad) {
            if (t == 0) *a.flag = 1;
            return;
        }
    }
    // R = R^ D (memory units), ||R^||_F^2
    double fr = 0.0;
    for (int j = warp; j < n; j += TC_NW) {
        const double dj = d[j] / a.sig_g;
        for (int i = lane; i < n; i += 32) {
            float v = 0.f;
            if (i <= j) {
                v = Tl[tc_idx(i >> 5, j >> 5) * TC_TILE + (i & 31) * TC_LD + (j & 31)];
                if (gmax <= 4e-6f && i == j) v = 1.0f;
                fr += (double)v * v;
            }
            a.R[i + (int64_t)j * a.ldr] = (float)((double)v * dj);
        }
    }
    __syncthreads();
    // the diagonal tiles of X replace those of R^ (not read by the inverse), freeing XD as scratch
    for (int e = t; e < nt * 1024; e += blockDim.x) {
        const int kb = e >> 10, i = (e >> 5) & 31, j = e & 31;
        Tl[tc_idx(kb, kb) * TC_TILE + i * TC_LD + j] = XD[kb * TC_TILE + i * TC_LD + j];
    }
    __syncthreads();
    // X = R^^-1 by block columns, left to right, in place of R^: X(ib, kb) = -[sum_{ib <= lb < kb}
    // X(ib, lb) R(lb, kb)] X_kk (column kb of R^ is dead once column kb of X is formed)
    if (gmax <= 4e-6f) {
        for (int e = t; e < nt * nt * 1024; e += blockDim.x) {
            const int tile = e >> 10, i = (e >> 5) & 31, j = e & 31;
            const int ib = tile % nt, jb = tile / nt;
            if (ib < jb) {
                float* p = Tl + tc_idx(ib, jb) * TC_TILE + i * TC_LD + j;
                *p = -*p;
            }
        }
    } else {
        for (int kb = 1; kb < nt; ++kb) {
            float c[4][4];
            if (task < kb) {   // T(ib) = sum_lb X(ib, lb) R(lb, kb), ib = task
                tc_zero(c);
                const int ib = task;
                for (int lb = ib; lb < kb; ++lb) {
                    tc_prod<false>(Tl + tc_idx(ib, lb) * TC_TILE, Tl + tc_idx(lb, kb) * TC_TILE, 0, 32, ti, tj, c);
                }
                tc_store(TMP + ib * TC_TILE, ti, tj, c, 1.0f);
            }
            __syncthreads();
            if (task < kb) {   // X(ib, kb) = -T(ib) X_kk
                tc_zero(c);
                tc_prod<false>(TMP + task * TC_TILE, Tl + tc_idx(kb, kb) * TC_TILE, 0, 32, ti, tj, c);
                tc_store(Tl + tc_idx(task, kb) * TC_TILE, ti, tj, c, -1.0f);
            }
            __syncthreads();
        }
    }
    // ||X||_F^2, max |X|
    double fx = 0.0;
    float mx = 0.f;
    for (int j = warp; j < n; j += TC_NW)
        for (int i = lane; i <= j; i += 32) {
            const float v = Tl[tc_idx(i >> 5, j >> 5) * TC_TILE + (i & 31) * TC_LD + (j & 31)];
            fx += (double)v * v;
            mx = fmaxf(mx, fabsf(v));
        }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        fr += __shfl_xor_sync(0xffffffffu, fr, o);
        fx += __shfl_xor_sync(0xffffffffu, fx, o);
        mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    if (lane == 0) {
        red[0][warp] = fr;
        red[1][warp] = fx;
        red[2][warp] = (double)mx;
    }
    __syncthreads();
    if (t < 32) {
        double a0 = t < TC_NW ? red[0][t] : 0.0, a1 = t < TC_NW ? red[1][t] : 0.0, m0 = t < TC_NW ? red[2][t] : 0.0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            a0 += __shfl_xor_sync(0xffffffffu, a0, o);
            a1 += __shfl_xor_sync(0xffffffffu, a1, o);
            m0 = fmax(m0, __shfl_xor_sync(0xffffffffu, m0, o));
        }
        if (t == 0) {
            red[0][0] = a0;
            red[1][0] = a1;
            red[2][0] = m0;
        }
    }
    __syncthreads();
    const double kap = sqrt(red[0][0] * red[1][0]);
    if (t == 0) a.kout[0] = kap;
    if (!(kap <= a.kappa_max)) {
        if (t == 0) *a.flag = 1;
        return;
    }
    // rho: R^^-1 into the fp16 range (largest entry in [2^14, 2^15))
    float rho = 1.0f;
    if (a.fp16) {
        int e;
        frexpf((float)red[2][0], &e);   // max in [2^(e-1), 2^e)
        rho = ldexpf(1.0f, 15 - e);
    }
    for (int idx = t; idx < TL_N * TL_N; idx += blockDim.x) {
        const int i = idx & (TL_N - 1), j = idx >> 8;
        a.rinv[idx] = (i <= j && j < n) ? Tl[tc_idx(i >> 5, j >> 5) * TC_TILE + (i & 31) * TC_LD + (j & 31)] * rho
                                        : 0.f;
    }
    for (int i = t; i < TL_N; i += blockDim.x) a.cscale[i] = i < n ? (float)((double)a.sig_a * a.sig_g * dinv[i]) : 0.f;
    if (t == 0) *a.escale = 1.0f / (a.sig_a * rho);
}

// ======================================================================= apply
struct TlApplyArgs {
    float* X;           // in place: X <- X R^-1 (fp32, ldx)
    int64_t ldx;
    int64_t m;
    int n;
    int vec;
    const float* rinv;  // [TL_N x TL_N] column-major R^^-1 (x rho)
    const float* cscale;
    const float* escale;
    const int* flag;    // nonzero: the Cholesky failed, leave X untouched
    int pf;             // L2 prefetch distance in the group's k-blocks (0: none)
};

// smem: B hi (TL_BBYTES) | B lo | TL_ASTAGES x (A hi 16 KB | A lo 16 KB) | cscale | barriers
constexpr int TL_AOFF = 2 * TL_BBYTES;
constexpr int TL_CSOFF = TL_AOFF + TL_ASTAGES * TL_ASTAGE;
constexpr int TL_BAROFF = TL_CSOFF + TL_N * 4;
constexpr int TL_APPLY_SMEM = TL_BAROFF + 128 + 1024;
constexpr int TL_GRAM_SMEM = TL_GSTAGES * TL_GSTAGE + 128 + 1024;
// first line of the K-block kc tile (lines j = 64 kc .. 255, one per output column)
__host__ __device__ constexpr int tl_btile(int kc) { return kc == 0 ? 0 : kc == 1 ? 256 : kc == 2 ? 448 : 576; }

constexpr int TL_ACW = 16;                               // apply converter warps 4..19 (two groups)
constexpr int TL_ATHREADS = 128 + 32 * TL_ACW + 128;   // + 4 epilogue warps (20..23)
template <bool BF>
__global__ void __launch_bounds__(TL_ATHREADS, 1) tl_apply_kernel(TlApplyArgs a) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    float* csc = reinterpret_cast<float*>(smem + TL_CSOFF);
    uint64_t* full_bar = reinterpret_cast<uint64_t*>(smem + TL_BAROFF);
    uint64_t* empty_bar = full_bar + TL_ASTAGES;
    uint64_t* tfull_bar = empty_bar + TL_ASTAGES;
    uint64_t* tempty_bar = tfull_bar + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty_bar + 2);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    RG_PDL_ENTRY();
    if (*a.flag) return;
    const int64_t ntiles = (a.m + 127) / 128;
    const int my = ntiles > blockIdx.x ? (int)((ntiles - 1 - blockIdx.x) / gridDim.x + 1) : 0;
    if (my == 0) return;

    if (threadIdx.x == 0) {
        for (int s = 0; s < TL_ASTAGES; ++s) {
            mbar_init(&full_bar[s], TL_ACW / 2);
            mbar_init(&empty_bar[s], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&tfull_bar[b], 1);
            mbar_init(&tempty_bar[b], 4);
        }
        fence_barrier_init();
    }
    if (warp == 1) tmem_alloc<512>(tmem_slot);
    // resident B: for K-block kc, line j (output column, j >= 64 kc) = R^^-1[64 kc .. 64 kc + 63][j]
    if (warp >= 4 && warp < 4 + TL_ACW) {
        const int cw = warp - 4, g = lane & 15;
        for (int L = 2 * cw + (lane >> 4); L < 640; L += 2 * TL_ACW) {
            const int kc = L < 256 ? 0 : L < 448 ? 1 : L < 576 ? 2 : 3;
            const int j = 64 * kc + (L - tl_btile(kc));
            float4 v = *reinterpret_cast<const float4*>(a.rinv + (int64_t)j * TL_N + 64 * kc + 4 * g);
            const uint32_t off = tl_swz(L, g);
            tl_split_sts<BF>(v, smem_u32(smem) + off, smem_u32(smem) + TL_BBYTES + off);
        }
        for (int i = threadIdx.x - 128; i < TL_N; i += 32 * TL_ACW) csc[i] = a.cscale[i];
        fence_proxy_async_smem();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (elect_one()) {
            // ---------------- MMA issuer: D[:, 64 kc ..] += A_kc B_kc (N = 256 - 64 kc), 3 split products
            const uint32_t b_hi = smem_u32(smem), b_lo = b_hi + TL_BBYTES;
            int it = 0;
            for (int tt = 0; tt < my; ++tt) {
                const int acc = tt & 1;
                mbar_wait(&tempty_bar[acc], ((uint32_t)(tt >> 1) & 1u) ^ 1u);
                tc_fence_after();
                const uint32_t d0 = tmem + acc * 256;
                for (int kc = 0; kc < 4; ++kc, ++it) {
                    const int s = it % TL_ASTAGES;
                    mbar_wait(&full_bar[s], (uint32_t)(it / TL_ASTAGES) & 1u);
                    tc_fence_after();
                    const uint32_t ah = smem_u32(smem + TL_AOFF + s * TL_ASTAGE), al = ah + TL_ASTAGE / 2;
                    const uint32_t N = 256 - 64 * kc;
                    const uint32_t idesc = umma_idesc_f16(128, N, 1u, 0u, BF ? 1u : 0u);
                    const uint32_t bh = b_hi + tl_btile(kc) * 128, bl = b_lo + tl_btile(kc) * 128;
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk) {
                        const uint64_t adh = umma_desc_sw128(ah + kk * 2048, 8192, 1024);
                        const uint64_t adl = umma_desc_sw128(al + kk * 2048, 8192, 1024);
                        const uint64_t bdh = umma_desc_sw128(bh + kk * 32, 16, 1024);
                        const uint64_t bdl = umma_desc_sw128(bl + kk * 32, 16, 1024);
                        const uint32_t accum = (kc > 0 || kk > 0) ? 1u : 0u;
                        umma_f16(d0 + 64 * kc, adh, bdh, idesc, accum);
                        umma_f16(d0 + 64 * kc, adh, bdl, idesc, 1u);
                        umma_f16(d0 + 64 * kc, adl, bdh, idesc, 1u);
                    }
                    umma_commit(&empty_bar[s]);
                }
                umma_commit(&tfull_bar[acc]);
            }
        }
        __syncwarp();
    } else if (warp >= 4 && warp < 4 + TL_ACW) {
        // ---------------- converters, two groups of 8 warps: group gr owns stage gr and converts
        // the k-blocks it = 4 tt + kc with it % 2 == gr, so one group's loads are in flight while
        // the other converts.  Line L = 2 pp + (lane >> 4): row half L >> 6, column 64 kc + (L & 63).
        const int gr = (warp - 4) >> 3, cw = (warp - 4) & 7, g = lane & 15;
        const int ti = 32 * cw + lane;   // 0..255 within the group
        for (int it = gr; it < 4 * my; it += 2) {
            const int tt = it >> 2, kc = it & 3;
            const int64_t t0 = ((int64_t)blockIdx.x + (int64_t)tt * gridDim.x) * 128;
            // the group's k-block pf steps ahead into L2, one 128 B line per thread (no registers held:
            // the register-staged loads alone keep ~64 KB per SM in flight; 1.31 -> 1.21 ms at config
            // 4 for pf = 1..3, slower from 4 on; 32 B-sector granularity was slower)
            if (a.pf > 0 && it + 2 * a.pf < 4 * my) {
                const int itp = it + 2 * a.pf;
                const int64_t tp = ((int64_t)blockIdx.x + (int64_t)(itp >> 2) * gridDim.x) * 128;
                const int c = 64 * (itp & 3) + (ti >> 2);
                const int64_t r = tp + 32 * (ti & 3);
                if (c < a.n && r < a.m) asm volatile("prefetch.global.L2 [%0];" ::"l"(a.X + (int64_t)c * a.ldx + r));
            }
            float4 v[8];
#pragma unroll
            for (int p = 0; p < 8; ++p) {
                const int L = 2 * (8 * cw + p) + (lane >> 4);
                const int c = 64 * kc + (L & 63);
                v[p] = c < a.n ? tl_load4(a.X + (int64_t)c * a.ldx, t0 + 64 * (L >> 6) + 4 * g, a.m, a.vec != 0)
                               : make_float4(0.f, 0.f, 0.f, 0.f);
            }
            mbar_wait(&empty_bar[gr], ((uint32_t)(it >> 1) & 1u) ^ 1u);
            uint8_t* ah = smem + TL_AOFF + gr * TL_ASTAGE;
#pragma unroll
            for (int p = 0; p < 8; ++p) {
                const int L = 2 * (8 * cw + p) + (lane >> 4);
                const float sc = csc[64 * kc + (L & 63)];
                float4 x = v[p];
                x.x *= sc; x.y *= sc; x.z *= sc; x.w *= sc;
                // MN-major: row half at +8 KB, line = column within the k-block
                const uint32_t off = tl_swz(L & 63, g) + (uint32_t)(L >> 6) * 8192u;
                tl_split_sts<BF>(x, smem_u32(ah) + off, smem_u32(ah) + TL_ASTAGE / 2 + off);
            }
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(&full_bar[gr]);
        }
    } else if (warp >= 4 + TL_ACW) {
        // ---------------- epilogue warps (TMEM lane quarter warp & 3): TMEM -> X in place.  A
        // tile's rows were all read (its four k-blocks converted) before its accumulator is full.
        const float es = *a.escale;
        const int q = warp & 3;
        for (int tt = 0; tt < my; ++tt) {
            const int64_t t0 = ((int64_t)blockIdx.x + (int64_t)tt * gridDim.x) * 128;
            const int acc = tt & 1;
            mbar_wait(&tfull_bar[acc], (uint32_t)(tt >> 1) & 1u);
            tc_fence_after();
            const int64_t row = t0 + 32 * q + lane;
#pragma unroll 1
            for (int c0 = 0; c0 < a.n; c0 += 32) {
                uint32_t r[32];
                tmem_ld32(tmem + acc * 256 + ((uint32_t)(32 * q) << 16) + c0, r);
                tmem_ld_wait();
                if (row < a.m) {
                    float* xp = a.X + row + (int64_t)c0 * a.ldx;
#pragma unroll
                    for (int j = 0; j < 32; ++j)
                        if (c0 + j < a.n) __stcs(xp + (int64_t)j * a.ldx, __uint_as_float(r[j]) * es);
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&tempty_bar[acc]);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1) tmem_dealloc<512>(tmem);
}

// ||I - G / sig^2||_F (fp64) of the Gram of a matrix with (near) unit columns: the exact
// orthogonality ||I - Q^T Q||_F in the Gram's precision (reading #33)
__global__ void __launch_bounds__(1024) tl_orth_kernel(const double* __restrict__ G, int n, double inv_s2, double* out) {
    RG_PDL_ENTRY();
    __shared__ double red[32];
    double acc = 0.0;
    for (int e = threadIdx.x; e < n * n; e += blockDim.x) {
        const int i = e % n, j = e / n;
        if (i > j) continue;
        const double v = G[e] * inv_s2 - (i == j ? 1.0 : 0.0);
        acc += (i == j ? 1.0 : 2.0) * v * v;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x < 32) {
        acc = red[threadIdx.x];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
        if (threadIdx.x == 0) *out = sqrt(acc);
    }
}
cudaError_t launch_tall_orth(const double* G, int n, double sig, double* out, cudaStream_t st) {
    RG_LAUNCH(tl_orth_kernel, 1, 1024, 0, st, G, n, 1.0 / (sig * sig), out);
    return cudaGetLastError();
}

// ======================================================================= launchers
size_t tall_ws_bytes() {
    return (size_t)TL_MAX_GRID * TL_PMAX * 4 + (size_t)TL_MAX_GRID * TL_N * 8 + (size_t)TL_N * TL_N * 8 +
           (size_t)TL_N * TL_N * 4 + TL_N * 4 + 128 + 64 + TL_N * 8;
}

double* tall_dbg(void* ws);
cudaError_t launch_tall_gram(const float* X, int64_t ldx, int64_t m, int n, float sig, int bf16, void* ws,
                             double* G, cudaStream_t st, const CUtensorMap* tmX) {
    uint8_t* w = reinterpret_cast<uint8_t*>(ws);
    float* part = reinterpret_cast<float*>(w);
    double* npart = reinterpret_cast<double*>(w + (size_t)TL_MAX_GRID * TL_PMAX * 4);
    const int64_t nchunks = (m + 63) / 64;
    const int grid = (int)std::min<int64_t>(std::min(dev_sms(), TL_MAX_GRID), std::max<int64_t>(nchunks, 1));
    TlGramArgs a{X, ldx, m, n, sig, ((reinterpret_cast<uintptr_t>(X) & 15) == 0 && (ldx & 3) == 0) ? 1 : 0, part,
                 npart};
    cudaError_t e;
    if (tmX && !getenv("RGSQR_TALL_NO_TMA")) {
        if (bf16) {
            if ((e = ensure_smem_attr((const void*)tl_gram_tma_kernel<true>, TL_GRAM_TMA_SMEM))) return e;
            RG_LAUNCH((tl_gram_tma_kernel<true>), grid, TL_TTHREADS, TL_GRAM_TMA_SMEM, st, *tmX, a);
        } else {
            if ((e = ensure_smem_attr((const void*)tl_gram_tma_kernel<false>, TL_GRAM_TMA_SMEM))) return e;
            RG_LAUNCH((tl_gram_tma_kernel<false>), grid, TL_TTHREADS, TL_GRAM_TMA_SMEM, st, *tmX, a);
        }
    } else if (bf16) {
        if ((e = ensure_smem_attr((const void*)tl_gram_kernel<true>, TL_GRAM_SMEM))) return e;
        RG_LAUNCH((tl_gram_kernel<true>), grid, TL_THREADS, TL_GRAM_SMEM, st, a);
    } else {
        if ((e = ensure_smem_attr((const void*)tl_gram_kernel<false>, TL_GRAM_SMEM))) return e;
        RG_LAUNCH((tl_gram_kernel<false>), grid, TL_THREADS, TL_GRAM_SMEM, st, a);
    }
    if (tmX && !getenv("RGSQR_TALL_NO_TMA")) {
        RG_LAUNCH(tl_reduce2_kernel, (TL_PART2 + TL_N + 255) / 256, 256, 0, st, part, npart, grid, n, G);
        RG_LAUNCH(tl_sym_kernel, dim3((n + 31) / 32, (n + 31) / 32), 1024, 0, st, G, n);
    } else {
        RG_LAUNCH(tl_reduce_kernel, (TL_PART + TL_N + 255) / 256, 256, 0, st, part, npart, grid, n, G,
                  getenv("RGSQR_TALL_DEBUG") ? tall_dbg(ws) : nullptr);
    }
    return cudaGetLastError();
}

// workspace tail: rinv [TL_N^2] fp32, cscale [TL_N], escale, flag, kout[2]
struct TallTail {
    float* rinv;
    float* cscale;
    float* escale;
    int* flag;
    double* kout;
};
static TallTail tall_tail(void* ws) {
    uint8_t* w = reinterpret_cast<uint8_t*>(ws) + (size_t)TL_MAX_GRID * TL_PMAX * 4 + (size_t)TL_MAX_GRID * TL_N * 8 +
                 (size_t)TL_N * TL_N * 8;
    TallTail t;
    t.rinv = reinterpret_cast<float*>(w);
    t.cscale = t.rinv + TL_N * TL_N;
    t.kout = reinterpret_cast<double*>(t.cscale + TL_N);
    t.escale = reinterpret_cast<float*>(t.kout + 4);   // kout: [kappa, pivot, orth, -]
    t.flag = reinterpret_cast<int*>(t.escale + 1);
    return t;
}
double* tall_gram_buffer(void* ws) {
    return reinterpret_cast<double*>(reinterpret_cast<uint8_t*>(ws) + (size_t)TL_MAX_GRID * TL_PMAX * 4 +
                                     (size_t)TL_MAX_GRID * TL_N * 8);
}
int* tall_flag(void* ws) { return tall_tail(ws).flag; }
double* tall_dbg(void* ws) { return tall_tail(ws).kout + 8; }
double* tall_kout(void* ws) { return tall_tail(ws).kout; }

constexpr int TL_CHOL_SMEM = (36 + TC_NT) * TC_TILE * 4 + 2 * TL_N * 8;

cudaError_t launch_tall_chol_apply(float* X, int64_t ldx, int64_t m, int n, const double* G, double sig_g, float sig_a,
                                   int bf16, double kappa_max, float* R, int64_t ldr, void* ws, cudaStream_t st) {
    TallTail t = tall_tail(ws);
    cudaError_t e;
    if ((e = cudaMemsetAsync(t.flag, 0, sizeof(int), st))) return e;
    TlCholArgs c{G, n, sig_g, sig_a, bf16 ? 0 : 1, kappa_max, R, ldr, t.rinv, t.cscale, t.escale, t.flag, t.kout};
    if ((e = ensure_smem_attr((const void*)tl_chol_kernel, TL_CHOL_SMEM))) return e;
    RG_LAUNCH(tl_chol_kernel, 1, TC_THREADS, TL_CHOL_SMEM, st, c);
    const int64_t ntiles = (m + 127) / 128;
    const int grid = (int)std::min<int64_t>(dev_sms(), std::max<int64_t>(ntiles, 1));
    TlApplyArgs a{X, ldx, m, n, ((reinterpret_cast<uintptr_t>(X) & 15) == 0 && (ldx & 3) == 0) ? 1 : 0,
                  t.rinv, t.cscale, t.escale, t.flag, 2};
    if (const char* s = getenv("RGSQR_TALL_PF")) a.pf = atoi(s);
    if (bf16) {
        if ((e = ensure_smem_attr((const void*)tl_apply_kernel<true>, TL_APPLY_SMEM))) return e;
        RG_LAUNCH((tl_apply_kernel<true>), grid, TL_ATHREADS, TL_APPLY_SMEM, st, a);
    } else {
        if ((e = ensure_smem_attr((const void*)tl_apply_kernel<false>, TL_APPLY_SMEM))) return e;
        RG_LAUNCH((tl_apply_kernel<false>), grid, TL_ATHREADS, TL_APPLY_SMEM, st, a);
    }
    return cudaGetLastError();
}

}  // namespace rg
