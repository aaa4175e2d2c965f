// gemm_tc.cu -- the two tensor-core contractions of Algorithm 1:
//
//   K1 projection  R12 = Q1^T A2        (line 8)   "TN": both operands K-major, K = m rows
//   K2 update      A2 <- A2 - Q1 R12    (line 9)   "NN": Q1 MN-major, R12 K-major, K = h
//
// fp16 (or bf16) operands, fp32 accumulation in TMEM (reading #3), issued
// with tcgen05.mma by one thread, operands staged by TMA into 128B-swizzled shared memory
// through an mbarrier ring.  K1 is split over m (deterministic two-stage reduction, no
// float atomics, reading #19); K2 fuses the fp32 read-modify-write of A2 and the fp16
// shadow write of the updated A2 into the TMEM epilogue.
//
// Split precision (reading #9, used by reorthogonalisation passes): each operand X is held
// as hi = fp16(X) and lo = fp16((X - hi) * 2^11); the kernels then issue three MMA groups
// hi*hi into accumulator 0 and hi*lo + lo*hi into accumulator 1 and combine
// D = D0 + D1 * 2^-11 in the epilogue.
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "kernels.h"
#include "ptx.cuh"

namespace rg {

constexpr int kBM = 128;    // UMMA M (rows of the accumulator = TMEM lanes)
constexpr int kBK = 64;     // k extent of one pipeline stage (one 128B swizzle row of fp16)
constexpr int kUK = 16;     // UMMA K for kind::f16
constexpr int kThreads = 128;

template <int BN, int STAGES, bool SPLIT>
struct GemmSmem {
    static constexpr int kABytes = kBM * kBK * 2;           // 16 KB
    static constexpr int kBBytes = BN * kBK * 2;
    static constexpr int kOps = SPLIT ? 2 : 1;               // hi (+ lo) copies of each operand
    static constexpr int kStageBytes = kOps * (kABytes + kBBytes);
    static constexpr int kDataBytes = STAGES * kStageBytes;
    static constexpr int kBarOffset = kDataBytes;
    static constexpr int kTotal = kDataBytes + 1024 /*barriers*/ + 1024 /*alignment slack*/;
};

template <int N>
struct TmemCols {
    static constexpr uint32_t value = N <= 32 ? 32 : N <= 64 ? 64 : N <= 128 ? 128 : N <= 256 ? 256 : 512;
};

struct GemmArgs {
    // K1 (projection): partial output P[z][j*ldp + i], K range in 64-row blocks
    float* P;
    int64_t ldp;           // leading dim of one partial (>= padded h)
    int64_t p_stride;      // elements between consecutive split partials
    int kb_total;          // ceil(m / 64)
    int kb_per_split;
    // K2 (update): C -= D over rows [0, m), cols [0, w)
    float* C;
    int64_t ldc;
    void* Ch;              // 16-bit shadow of the updated C (hi part), may be null
    void* Cl;              // 16-bit lo part (split mode), may be null
    int64_t ldh;
    int64_t m;
    int w;
    int kb_h;              // ceil(h / 64)
    int bf16;
};

__device__ __forceinline__ uint16_t f2h_bits(float x, int bf16) {
    if (bf16) {
        __nv_bfloat16 b = __float2bfloat16_rn(x);
        return *reinterpret_cast<uint16_t*>(&b);
    }
    __half h = __float2half_rn(x);
    return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float h2f_bits(uint16_t u, int bf16) {
    if (bf16) {
        __nv_bfloat16 b = *reinterpret_cast<__nv_bfloat16*>(&u);
        return __bfloat162float(b);
    }
    __half h = *reinterpret_cast<__half*>(&u);
    return __half2float(h);
}

// MODE 0 = K1 projection (A, B K-major; grid = (tiles_i, tiles_j, splits))
// MODE 1 = K2 update     (A MN-major, B K-major; grid = (row tiles, col tiles))
template <int MODE, int BN, int STAGES, bool SPLIT>
__global__ void __launch_bounds__(kThreads, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ CUtensorMap tmA_lo, const __grid_constant__ CUtensorMap tmB_lo,
                   GemmArgs args) {
    using L = GemmSmem<BN, STAGES, SPLIT>;
    constexpr uint32_t kTmemCols = TmemCols<(SPLIT ? 2 : 1) * BN>::value;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint64_t* full_bar = reinterpret_cast<uint64_t*>(smem + L::kBarOffset);
    uint64_t* empty_bar = full_bar + STAGES;
    uint64_t* accum_bar = empty_bar + STAGES;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(accum_bar + 1);

    const int warp = threadIdx.x >> 5;
    int kb_begin, kb_end;
    if (MODE == 0) {
        kb_begin = blockIdx.z * args.kb_per_split;
        kb_end = min(kb_begin + args.kb_per_split, args.kb_total);
    } else {
        kb_begin = 0;
        kb_end = args.kb_h;
    }
    const int tile0 = blockIdx.x * kBM;   // i (K1: Q1 column) or r (K2: row)
    const int tile1 = blockIdx.y * BN;    // j (A2 column)

    if (threadIdx.x == 0) {
        tma_prefetch_desc(&tmA);
        tma_prefetch_desc(&tmB);
        if (SPLIT) {
            tma_prefetch_desc(&tmA_lo);
            tma_prefetch_desc(&tmB_lo);
        }
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&full_bar[s], 1);
            mbar_init(&empty_bar[s], 1);
        }
        mbar_init(accum_bar, 1);
        fence_barrier_init();
    }
    if (warp == 2) tmem_alloc<kTmemCols>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0 && elect_one()) {
        // ---------------- TMA producer
        for (int kb = kb_begin; kb < kb_end; ++kb) {
            const int it = kb - kb_begin;
            const int s = it % STAGES;
            const uint32_t round = it / STAGES;
            mbar_wait(&empty_bar[s], (round & 1u) ^ 1u);
            uint8_t* sa = smem + s * L::kStageBytes;
            uint8_t* sb = sa + L::kABytes;
            mbar_arrive_expect_tx(&full_bar[s], L::kStageBytes);
            if (MODE == 0) {
                tma_load_2d(sa, &tmA, &full_bar[s], kb * kBK, tile0);
                tma_load_2d(sb, &tmB, &full_bar[s], kb * kBK, tile1);
                if (SPLIT) {
                    tma_load_2d(sb + L::kBBytes, &tmA_lo, &full_bar[s], kb * kBK, tile0);
                    tma_load_2d(sb + L::kBBytes + L::kABytes, &tmB_lo, &full_bar[s], kb * kBK, tile1);
                }
            } else {
                // MN-major A: two 64(row) x 64(k) boxes, the second at +8 KB (LBO)
                tma_load_2d(sa, &tmA, &full_bar[s], tile0, kb * kBK);
                tma_load_2d(sa + L::kABytes / 2, &tmA, &full_bar[s], tile0 + 64, kb * kBK);
                tma_load_2d(sb, &tmB, &full_bar[s], kb * kBK, tile1);
                if (SPLIT) {
                    uint8_t* sal = sb + L::kBBytes;
                    tma_load_2d(sal, &tmA_lo, &full_bar[s], tile0, kb * kBK);
                    tma_load_2d(sal + L::kABytes / 2, &tmA_lo, &full_bar[s], tile0 + 64, kb * kBK);
                    tma_load_2d(sal + L::kABytes, &tmB_lo, &full_bar[s], kb * kBK, tile1);
                }
            }
        }
    } else if (warp == 1 && elect_one()) {
        // ---------------- MMA issuer (single thread)
        const uint32_t idesc = umma_idesc_f16(kBM, BN, MODE == 1 ? 1u : 0u, 0u, (uint32_t)args.bf16);
        for (int kb = kb_begin; kb < kb_end; ++kb) {
            const int it = kb - kb_begin;
            const int s = it % STAGES;
            const uint32_t round = it / STAGES;
            mbar_wait(&full_bar[s], round & 1u);
            tc_fence_after();
            const uint32_t sa = smem_u32(smem + s * L::kStageBytes);
            const uint32_t sb = sa + L::kABytes;
            const uint32_t sal = sb + L::kBBytes;
            const uint32_t sbl = sal + L::kABytes;
#pragma unroll
            for (int kk = 0; kk < kBK / kUK; ++kk) {
                uint64_t ad, adl;
                if (MODE == 0) {
                    ad = umma_desc_sw128(sa + kk * 32, 16, 1024);
                    adl = umma_desc_sw128(sal + kk * 32, 16, 1024);
                } else {
                    ad = umma_desc_sw128(sa + kk * 2048, L::kABytes / 2, 1024);
                    adl = umma_desc_sw128(sal + kk * 2048, L::kABytes / 2, 1024);
                }
                const uint64_t bd = umma_desc_sw128(sb + kk * 32, 16, 1024);
                const uint32_t acc = (it > 0 || kk > 0) ? 1u : 0u;
                umma_f16(tmem_base, ad, bd, idesc, acc);
                if (SPLIT) {
                    const uint64_t bdl = umma_desc_sw128(sbl + kk * 32, 16, 1024);
                    umma_f16(tmem_base + BN, ad, bdl, idesc, acc);   // hi * lo
                    umma_f16(tmem_base + BN, adl, bd, idesc, 1u);    // lo * hi
                }
            }
            umma_commit(&empty_bar[s]);
        }
        umma_commit(accum_bar);
    }

    // ---------------- epilogue: all 4 warps, thread <-> accumulator row (TMEM lane)
    __syncwarp();
    mbar_wait(accum_bar, 0);
    tc_fence_after();
    const int row = warp * 32 + (threadIdx.x & 31);
    const uint32_t lane_addr = tmem_base + (static_cast<uint32_t>(warp * 32) << 16);
    const bool empty_range = kb_end <= kb_begin;
#pragma unroll 1
    for (int c = 0; c < BN; c += 32) {
        uint32_t v[32];
        tmem_ld32(lane_addr + c, v);
        float d[32];
        tmem_ld_wait();
#pragma unroll
        for (int jj = 0; jj < 32; ++jj) d[jj] = empty_range ? 0.f : __uint_as_float(v[jj]);
        if (SPLIT) {
            uint32_t u[32];
            tmem_ld32(lane_addr + BN + c, u);
            tmem_ld_wait();
#pragma unroll
            for (int jj = 0; jj < 32; ++jj)
                d[jj] += empty_range ? 0.f : __uint_as_float(u[jj]) * (1.0f / 2048.0f);
        }
        if (MODE == 0) {
            float* out = args.P + blockIdx.z * args.p_stride + (int64_t)(tile1 + c) * args.ldp + tile0 + row;
#pragma unroll
            for (int jj = 0; jj < 32; ++jj) out[(int64_t)jj * args.ldp] = d[jj];
        } else {
            const int64_t r = (int64_t)tile0 + row;
            if (r < args.m) {
                float* cp = args.C + r;
                float old[32];
#pragma unroll
                for (int jj = 0; jj < 32; ++jj) {
                    const int j = tile1 + c + jj;
                    old[jj] = (j < args.w) ? cp[(int64_t)j * args.ldc] : 0.f;
                }
#pragma unroll
                for (int jj = 0; jj < 32; ++jj) {
                    const int j = tile1 + c + jj;
                    if (j < args.w) {
                        const float nv = old[jj] - d[jj];
                        cp[(int64_t)j * args.ldc] = nv;
                        if (args.Ch) {
                            const uint16_t hb = f2h_bits(nv, args.bf16);
                            reinterpret_cast<uint16_t*>(args.Ch)[r + (int64_t)j * args.ldh] = hb;
                            if (args.Cl) {
                                const float lo = (nv - h2f_bits(hb, args.bf16)) * 2048.0f;
                                reinterpret_cast<uint16_t*>(args.Cl)[r + (int64_t)j * args.ldh] =
                                    f2h_bits(lo, args.bf16);
                            }
                        }
                    }
                }
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) tmem_dealloc<kTmemCols>(tmem_base);
}

// --------------------------------------------------------------------------------------
// split-K reduction for K1: R12(i,j) = sum_z P[z](i,j) in fixed z order (deterministic),
// written as fp32 into R (ldr) and rounded to 16 bit (hi, and lo for split mode) into
// the K2 B-operand image R12h (K-major: column j holds R12(:, j), ld = ldh).
__global__ void __launch_bounds__(256) proj_reduce_kernel(const float* __restrict__ P, int64_t ldp, int64_t p_stride,
                                                          int splits, int h, int w, float* __restrict__ R, int64_t ldr,
                                                          float* __restrict__ Rf, int64_t ldf, uint16_t* __restrict__ Rh,
                                                          uint16_t* __restrict__ Rl, int64_t ldh, int bf16) {
    // block (32, 8): 32 consecutive outputs x 8 split lanes; lane ty sums splits ty, ty+8, ...
    // in order, then the 8 lane sums are added in order (deterministic).
    __shared__ float part[8][33];
    const int64_t total = (int64_t)h * w;
    const int64_t e = (int64_t)blockIdx.x * 32 + threadIdx.x;
    const bool valid = e < total;
    const int i = valid ? (int)(e % h) : 0;
    const int j = valid ? (int)(e / h) : 0;
    const float* p = P + (int64_t)j * ldp + i;
    float s = 0.f;
    if (valid) {
        int z = threadIdx.y;
        for (; z + 24 < splits; z += 32) {
            const float a = __ldcg(p + (int64_t)z * p_stride), b = __ldcg(p + (int64_t)(z + 8) * p_stride);
            const float c = __ldcg(p + (int64_t)(z + 16) * p_stride), d = __ldcg(p + (int64_t)(z + 24) * p_stride);
            s += a; s += b; s += c; s += d;
        }
        for (; z < splits; z += 8) s += __ldcg(p + (int64_t)z * p_stride);
    }
    part[threadIdx.y][threadIdx.x] = s;
    __syncthreads();
    if (threadIdx.y != 0 || !valid) return;
    float t = 0.f;
#pragma unroll
    for (int y = 0; y < 8; ++y) t += part[y][threadIdx.x];
    if (R) R[i + (int64_t)j * ldr] = t;
    if (Rf) Rf[i + (int64_t)j * ldf] = t;
    if (Rh) {
        const uint16_t hb = f2h_bits(t, bf16);
        Rh[i + (int64_t)j * ldh] = hb;
        if (Rl) Rl[i + (int64_t)j * ldh] = f2h_bits((t - h2f_bits(hb, bf16)) * 2048.0f, bf16);
    }
}

// After a cross-rank allreduce of Rf: write R and the 16-bit images.
__global__ void proj_finish_kernel(const float* __restrict__ Rf, int64_t ldf, int h, int w, float* __restrict__ R,
                                   int64_t ldr, uint16_t* __restrict__ Rh, uint16_t* __restrict__ Rl, int64_t ldh,
                                   int bf16) {
    const int64_t total = (int64_t)h * w;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int i = (int)(e % h);
        const int j = (int)(e / h);
        const float s = Rf[i + (int64_t)j * ldf];
        R[i + (int64_t)j * ldr] = s;
        const uint16_t hb = f2h_bits(s, bf16);
        Rh[i + (int64_t)j * ldh] = hb;
        if (Rl) Rl[i + (int64_t)j * ldh] = f2h_bits((s - h2f_bits(hb, bf16)) * 2048.0f, bf16);
    }
}

// ------------------------------------------------------------------ host launchers
template <int MODE, int BN, int STAGES, bool SPLIT>
static cudaError_t launch_gemm(dim3 grid, const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& al,
                               const CUtensorMap& bl, const GemmArgs& args, cudaStream_t st) {
    using L = GemmSmem<BN, STAGES, SPLIT>;
    auto kern = gemm_tc_kernel<MODE, BN, STAGES, SPLIT>;
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, L::kTotal);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    ++g_launches;
    kern<<<grid, kThreads, L::kTotal, st>>>(a, b, al, bl, args);
    return cudaGetLastError();
}

template <int MODE, bool SPLIT>
static cudaError_t dispatch_bn(int bn, dim3 grid, const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& al,
                               const CUtensorMap& bl, const GemmArgs& args, cudaStream_t st) {
    // stage counts keep smem <= ~200 KB: (16 KB + BN*128 B) * ops * stages
    switch (bn) {
        case 32: return launch_gemm<MODE, 32, SPLIT ? 4 : 6, SPLIT>(grid, a, b, al, bl, args, st);
        case 64: return launch_gemm<MODE, 64, SPLIT ? 4 : 6, SPLIT>(grid, a, b, al, bl, args, st);
        case 128: return launch_gemm<MODE, 128, SPLIT ? 3 : 5, SPLIT>(grid, a, b, al, bl, args, st);
        case 256: return launch_gemm<MODE, 256, SPLIT ? 2 : 4, SPLIT>(grid, a, b, al, bl, args, st);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_proj_gemm(int bn, bool split, int tiles_i, int tiles_j, int splits, const CUtensorMap& q1,
                             const CUtensorMap& a2, const CUtensorMap& q1_lo, const CUtensorMap& a2_lo, float* P,
                             int64_t ldp, int64_t p_stride, int kb_total, int kb_per_split, int bf16,
                             cudaStream_t st) {
    GemmArgs args{};
    args.P = P;
    args.ldp = ldp;
    args.p_stride = p_stride;
    args.kb_total = kb_total;
    args.kb_per_split = kb_per_split;
    args.bf16 = bf16;
    dim3 grid(tiles_i, tiles_j, splits);
    return split ? dispatch_bn<0, true>(bn, grid, q1, a2, q1_lo, a2_lo, args, st)
                 : dispatch_bn<0, false>(bn, grid, q1, a2, q1, a2, args, st);
}

cudaError_t launch_update_gemm(int bn, bool split, int64_t m, int w, int h, const CUtensorMap& q1_mn,
                               const CUtensorMap& r12, const CUtensorMap& q1_mn_lo, const CUtensorMap& r12_lo,
                               float* C, int64_t ldc, void* Ch, void* Cl, int64_t ldh, int bf16, cudaStream_t st) {
    GemmArgs args{};
    args.C = C;
    args.ldc = ldc;
    args.Ch = Ch;
    args.Cl = Cl;
    args.ldh = ldh;
    args.m = m;
    args.w = w;
    args.kb_h = (h + kBK - 1) / kBK;
    args.bf16 = bf16;
    dim3 grid((unsigned)((m + kBM - 1) / kBM), (unsigned)((w + bn - 1) / bn), 1);
    return split ? dispatch_bn<1, true>(bn, grid, q1_mn, r12, q1_mn_lo, r12_lo, args, st)
                 : dispatch_bn<1, false>(bn, grid, q1_mn, r12, q1_mn, r12, args, st);
}

cudaError_t launch_proj_reduce(const float* P, int64_t ldp, int64_t p_stride, int splits, int h, int w, float* R,
                               int64_t ldr, float* Rf, int64_t ldf, uint16_t* Rh, uint16_t* Rl, int64_t ldh, int bf16,
                               cudaStream_t st) {
    const int64_t total = (int64_t)h * w;
    ++g_launches;
    proj_reduce_kernel<<<(unsigned)((total + 31) / 32), dim3(32, 8), 0, st>>>(P, ldp, p_stride, splits, h, w, R, ldr,
                                                                              Rf, ldf, Rh, Rl, ldh, bf16);
    return cudaGetLastError();
}

cudaError_t launch_proj_finish(const float* Rf, int64_t ldf, int h, int w, float* R, int64_t ldr, uint16_t* Rh,
                               uint16_t* Rl, int64_t ldh, int bf16, cudaStream_t st) {
    const int64_t total = (int64_t)h * w;
    int blocks = (int)((total + 255) / 256);
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    ++g_launches;
    proj_finish_kernel<<<blocks, 256, 0, st>>>(Rf, ldf, h, w, R, ldr, Rh, Rl, ldh, bf16);
    return cudaGetLastError();
}

}  // namespace rg
