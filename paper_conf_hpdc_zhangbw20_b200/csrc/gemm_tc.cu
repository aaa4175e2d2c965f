// gemm_tc.cu -- the two tensor-core contractions of Algorithm 1:
//
//   K1 projection  R12 = Q1^T A2        (line 8)   "TN": both operands K-major, K = m rows
//   K2 update      A2 <- A2 - Q1 R12    (line 9)   "NN": Q1 MN-major, R12 K-major, K = h
//
// fp16 (or bf16) operands, fp32 accumulation in TMEM (reading #3), issued
// with tcgen05.mma by one thread, operands staged by TMA into 128B-swizzled shared memory
// through an mbarrier ring.  Persistent, warp-specialised kernel:
//   warp 0      TMA producer            warp 1   MMA issuer (one elected lane)
//   warp 2      TMEM allocator          warp 3   idle
//   warps 4..   epilogue warpgroup(s): TMEM -> registers -> per-warp smem transpose ->
//               16-byte global accesses (4 consecutive rows of one column per lane)
// Two TMEM accumulator buffers (when they fit) let the epilogue of one tile overlap the
// MMAs of the next.  K1 is split over m with a deterministic two-stage reduction (no float
// atomics, reading #19); K2 fuses the fp32 read-modify-write of A2 and the 16-bit shadow
// write of the updated A2 into the epilogue.
//
// Split precision (reading #9, reorthogonalisation passes): operands are held as
// hi = fp16(X) and lo = fp16((X - hi) 2^11); three MMA groups accumulate hi*hi into
// accumulator 0 and hi*lo + lo*hi into accumulator 1; D = D0 + 2^-11 D1 in the epilogue.
#include <cstdlib>

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
constexpr int kEpiLd = 36;  // per-warp transpose buffer row stride (floats, 16B aligned)

// TE = number of C chunk slots (128 rows x 32 columns, fp32) of the TMA epilogue, split evenly
// between the epilogue warpgroups; 0 = register epilogue
template <int BN, int STAGES, bool SPLIT, int EPI_WG, int TE = 0>
struct GemmCfg {
    static constexpr int kABytes = kBM * kBK * 2;           // 16 KB
    static constexpr int kBBytes = BN * kBK * 2;
    static constexpr int kOps = SPLIT ? 2 : 1;               // hi (+ lo) copies of each operand
    static constexpr int kStageBytes = kOps * (kABytes + kBBytes);
    static constexpr int kDataBytes = STAGES * kStageBytes;
    static constexpr int kEpiWarps = 4 * EPI_WG;
    static constexpr int kCSlot = kBM * 32 * 4;               // fp32 C chunk, [32 cols][128 rows]
    static constexpr int kEpiBytes = TE ? TE * kCSlot : kEpiWarps * 32 * kEpiLd * 4;
    static constexpr int kBarOffset = kDataBytes + kEpiBytes;
    static constexpr int kTotal = kBarOffset + 512 + 1024;   // barriers + 1 KB alignment slack
    static constexpr int kThreads = 128 + 32 * kEpiWarps;
    static constexpr int kAccCols = SPLIT ? 2 * BN : BN;
    static constexpr int kAcc = (2 * kAccCols <= 512) ? 2 : 1;  // TMEM accumulator buffers
    static constexpr uint32_t kTmemCols = (kAcc * kAccCols <= 32) ? 32 : (kAcc * kAccCols <= 64) ? 64
                                        : (kAcc * kAccCols <= 128) ? 128 : (kAcc * kAccCols <= 256) ? 256 : 512;
};

struct GemmArgs {
    // work decomposition
    int units;             // total work units
    int tiles_i, tiles_j;  // output tiles (MODE 0: i = Q1 col tiles; MODE 1: i = row tiles)
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
    int vec_ok;            // C / Ch / Cl accesses may use 16-byte (8-byte) vectors
    int overwrite;         // K2 only: C = D instead of C -= D (plain product, lowrank_approx)
    int h0;                // K2 only: 16-bit image written for columns >= h0 only
    int c_ef;              // K2 TMA epilogue: C read / written with the L2 evict_first policy (streamed
                           // once; keeps the next leaf's code and operands resident)
    int jfast;             // K1: units enumerate the N tiles fastest (A is the operand too large for L2)
    int mc;                // K2: cluster pair along M sharing the B tile (TMA multicast of its halves);
                           // units are pair units, CTA rank blockIdx.x & 1 takes row block 2 (u / tiles_j) + rank
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

// unit -> (t0 = first row of the M tile, tj = N tile index, z = split, [kb0, kb1))
template <int MODE>
__device__ __forceinline__ void unit_coords(const GemmArgs& a, int u, int& t0, int& tj, int& z, int& kb0, int& kb1) {
    if (MODE == 0) {
        const int tiles = a.tiles_i * a.tiles_j;
        z = u / tiles;
        const int rem = u % tiles;
        if (a.jfast) {   // N tiles fastest: the concurrent CTAs share one A tile (read once from HBM)
            t0 = (rem / a.tiles_j) * kBM;
            tj = rem % a.tiles_j;
        } else {          // M tiles fastest: the concurrent CTAs share one B tile
            t0 = (rem % a.tiles_i) * kBM;
            tj = rem / a.tiles_i;
        }
        kb0 = z * a.kb_per_split;
        kb1 = min(kb0 + a.kb_per_split, a.kb_total);
    } else {
        z = 0;
        t0 = (a.mc ? 2 * (u / a.tiles_j) + (int)(blockIdx.x & 1) : u / a.tiles_j) * kBM;
        tj = u % a.tiles_j;
        kb0 = 0;
        kb1 = a.kb_h;
    }
}

// MODE 0 = K1 projection (A, B K-major), MODE 1 = K2 update (A MN-major, B K-major)
// TMA-epilogue slot of chunk ch of the cnt-th tile of this CTA: warpgroup g = ch % EPI_WG owns
// slots [g * NCW, (g + 1) * NCW) and fills them round-robin in its own chunk order.
template <int KCH, int EPI_WG, int NCW>
__device__ __forceinline__ void te_slot(int cnt, int ch, int& s, uint32_t& round) {
    const int g = ch % EPI_WG;
    const int per = (KCH - g + EPI_WG - 1) / EPI_WG;   // chunks per tile of warpgroup g
    const int k = cnt * per + ch / EPI_WG;
    s = g * NCW + k % NCW;
    round = (uint32_t)(k / NCW);
}

// TE (K2 only): TMA epilogue.  Warp 3 streams the fp32 C chunks (128 rows x 32 columns, 16 KB)
// of the tiles into per-warpgroup rings of shared-memory slots ahead of the accumulators; each
// epilogue warp subtracts its TMEM rows from the slot in place (and stores the 16-bit image of
// its rows directly, 64 contiguous bytes per column and warp); warp 2 (idle after the TMEM
// allocation) issues the TMA stores and recycles the slots.  Several C chunks per SM are in
// flight (the register-staged epilogue kept one chunk ahead and reached ~3.5-4 TB/s on the
// HBM-bound levels).
template <int MODE, int BN, int STAGES, bool SPLIT, int EPI_WG, int TE = 0>
__global__ void __launch_bounds__(GemmCfg<BN, STAGES, SPLIT, EPI_WG, TE>::kThreads, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ CUtensorMap tmA_lo, const __grid_constant__ CUtensorMap tmB_lo,
                   const __grid_constant__ CUtensorMap tmC, GemmArgs args) {
    using C = GemmCfg<BN, STAGES, SPLIT, EPI_WG, TE>;
    static_assert(!TE || (MODE == 1 && !SPLIT), "TMA epilogue: K2, single precision");
    // Chunk ch of a tile belongs to warpgroup ch % EPI_WG, which owns TE / EPI_WG slots and uses
    // them round-robin in its own chunk order, so every slot has one consumer that waits its
    // rounds in order.  (A ring shared by both warpgroups lets one wait on round r + 1 of a slot
    // while the other's round r -- a TMA load completing out of order -- is still pending:
    // mbarrier parity aliasing, measured as sporadic hangs / launch failures.)
    static_assert(TE % EPI_WG == 0, "C ring slots split evenly between the epilogue warpgroups");
    constexpr int kNcw = TE > 0 ? TE / EPI_WG : 1;   // slots per warpgroup
    constexpr int kCRing = TE > 0 ? TE : 1;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    float* epi_buf = reinterpret_cast<float*>(smem + C::kDataBytes);
    uint64_t* full_bar = reinterpret_cast<uint64_t*>(smem + C::kBarOffset);
    uint64_t* empty_bar = full_bar + STAGES;
    uint64_t* tfull_bar = empty_bar + STAGES;
    uint64_t* tempty_bar = tfull_bar + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty_bar + 2);
    uint64_t* cfull_bar = reinterpret_cast<uint64_t*>(smem + C::kBarOffset + 256);
    uint64_t* cempty_bar = cfull_bar + kCRing;
    uint64_t* cready_bar = cempty_bar + kCRing;

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;

    if (threadIdx.x == 0) {
        tma_prefetch_desc(&tmA);
        tma_prefetch_desc(&tmB);
        if (SPLIT) {
            tma_prefetch_desc(&tmA_lo);
            tma_prefetch_desc(&tmB_lo);
        }
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&full_bar[s], 1);
            mbar_init(&empty_bar[s], args.mc ? 2 : 1);   // both CTAs of a pair read every B stage
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&tfull_bar[a], 1);
            mbar_init(&tempty_bar[a], C::kEpiWarps);
        }
        if (TE) {
            for (int s = 0; s < kCRing; ++s) {
                mbar_init(&cfull_bar[s], 1);
                mbar_init(&cempty_bar[s], 1);
                mbar_init(&cready_bar[s], 4);   // the four warps of the epilogue warpgroup
            }
            tma_prefetch_desc(&tmC);
        }
        fence_barrier_init();
    }
    if (warp == 2) tmem_alloc<C::kTmemCols>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    if (args.mc) cluster_sync_all();   // the peer's barriers are initialised before any multicast
    RG_PDL_ENTRY();   // prologue above overlaps the previous kernel's tail
    const int ubeg = args.mc ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
    const int ustep = args.mc ? (int)(gridDim.x >> 1) : (int)gridDim.x;

    if (warp == 0) {
        if (elect_one()) {
            // ---------------- TMA producer
            int it = 0;
            for (int u = ubeg; u < args.units; u += ustep) {
                int t0, tj, z, kb0, kb1;
                unit_coords<MODE>(args, u, t0, tj, z, kb0, kb1);
                const int t1 = tj * BN;
                for (int kb = kb0; kb < kb1; ++kb, ++it) {
                    const int s = it % STAGES;
                    const uint32_t round = it / STAGES;
                    mbar_wait(&empty_bar[s], (round & 1u) ^ 1u);
                    uint8_t* sa = smem + s * C::kStageBytes;
                    uint8_t* sb = sa + C::kABytes;
                    mbar_arrive_expect_tx(&full_bar[s], C::kStageBytes);
                    if (MODE == 0) {
                        tma_load_2d(sa, &tmA, &full_bar[s], kb * kBK, t0);
                        tma_load_2d(sb, &tmB, &full_bar[s], kb * kBK, t1);
                        if (SPLIT) {
                            tma_load_2d(sb + C::kBBytes, &tmA_lo, &full_bar[s], kb * kBK, t0);
                            tma_load_2d(sb + C::kBBytes + C::kABytes, &tmB_lo, &full_bar[s], kb * kBK, t1);
                        }
                    } else {
                        // MN-major A: two 64(row) x 64(k) boxes, the second at +8 KB (LBO)
                        tma_load_2d(sa, &tmA, &full_bar[s], t0, kb * kBK);
                        tma_load_2d(sa + C::kABytes / 2, &tmA, &full_bar[s], t0 + 64, kb * kBK);
                        if (!SPLIT && args.mc) {   // this CTA's half of the B tile, into both CTAs of the pair
                            const int rk = (int)(blockIdx.x & 1);
                            tma_load_2d_mc(sb + rk * (C::kBBytes / 2), &tmB_lo, &full_bar[s], kb * kBK,
                                           t1 + rk * (BN / 2), (uint16_t)3);
                        } else {
                            tma_load_2d(sb, &tmB, &full_bar[s], kb * kBK, t1);
                        }
                        if (SPLIT) {
                            uint8_t* sal = sb + C::kBBytes;
                            tma_load_2d(sal, &tmA_lo, &full_bar[s], t0, kb * kBK);
                            tma_load_2d(sal + C::kABytes / 2, &tmA_lo, &full_bar[s], t0 + 64, kb * kBK);
                            tma_load_2d(sal + C::kABytes, &tmB_lo, &full_bar[s], kb * kBK, t1);
                        }
                    }
                }
            }
        }
        __syncwarp();
    } else if (warp == 1) {
        if (elect_one()) {
            // ---------------- MMA issuer (single thread)
            const uint32_t idesc = umma_idesc_f16(kBM, BN, MODE == 1 ? 1u : 0u, 0u, (uint32_t)args.bf16);
            int it = 0, cnt = 0;
            for (int u = ubeg; u < args.units; u += ustep, ++cnt) {
                int t0, tj, z, kb0, kb1;
                unit_coords<MODE>(args, u, t0, tj, z, kb0, kb1);
                const int acc = cnt % C::kAcc;
                const uint32_t aphase = (uint32_t)(cnt / C::kAcc) & 1u;
                mbar_wait(&tempty_bar[acc], aphase ^ 1u);
                tc_fence_after();
                const uint32_t dtm = tmem_base + acc * C::kAccCols;
                for (int kb = kb0; kb < kb1; ++kb, ++it) {
                    const int s = it % STAGES;
                    const uint32_t round = it / STAGES;
                    mbar_wait(&full_bar[s], round & 1u);
                    tc_fence_after();
                    const uint32_t sa = smem_u32(smem + s * C::kStageBytes);
                    const uint32_t sb = sa + C::kABytes;
                    const uint32_t sal = sb + C::kBBytes;
                    const uint32_t sbl = sal + C::kABytes;
#pragma unroll
                    for (int kk = 0; kk < kBK / kUK; ++kk) {
                        uint64_t ad, adl;
                        if (MODE == 0) {
                            ad = umma_desc_sw128(sa + kk * 32, 16, 1024);
                            adl = umma_desc_sw128(sal + kk * 32, 16, 1024);
                        } else {
                            ad = umma_desc_sw128(sa + kk * 2048, C::kABytes / 2, 1024);
                            adl = umma_desc_sw128(sal + kk * 2048, C::kABytes / 2, 1024);
                        }
                        const uint64_t bd = umma_desc_sw128(sb + kk * 32, 16, 1024);
                        const uint32_t accum = (kb > kb0 || kk > 0) ? 1u : 0u;
                        umma_f16(dtm, ad, bd, idesc, accum);
                        if (SPLIT) {
                            const uint64_t bdl = umma_desc_sw128(sbl + kk * 32, 16, 1024);
                            umma_f16(dtm + BN, ad, bdl, idesc, accum);   // hi * lo
                            umma_f16(dtm + BN, adl, bd, idesc, 1u);      // lo * hi
                        }
                    }
                    if (args.mc) umma_commit_mc(&empty_bar[s], (uint16_t)3);
                    else umma_commit(&empty_bar[s]);
                }
                umma_commit(&tfull_bar[acc]);
            }
        }
        __syncwarp();
    } else if (TE && warp == 3) {
        if (elect_one()) {
            // ---------------- C producer: fp32 C chunks into the slot ring (chunk order = t)
            constexpr int kChunks = BN / 32;
            int cnt = 0;
            for (int u = ubeg; u < args.units; u += ustep, ++cnt) {
                int t0, tj, z, kb0, kb1;
                unit_coords<MODE>(args, u, t0, tj, z, kb0, kb1);
                for (int ch = 0; ch < kChunks; ++ch) {
                    int s;
                    uint32_t round;
                    te_slot<kChunks, EPI_WG, kNcw>(cnt, ch, s, round);
                    mbar_wait(&cempty_bar[s], (round & 1u) ^ 1u);
                    if (args.overwrite) {
                        mbar_arrive(&cfull_bar[s]);
                    } else {
                        mbar_arrive_expect_tx(&cfull_bar[s], C::kCSlot);
                        if (args.c_ef)
                            tma_load_2d_hint(epi_buf + s * (C::kCSlot / 4), &tmC, &cfull_bar[s], t0, tj * BN + ch * 32,
                                             policy_evict_first());
                        else
                            tma_load_2d(epi_buf + s * (C::kCSlot / 4), &tmC, &cfull_bar[s], t0, tj * BN + ch * 32);
                    }
                }
            }
        }
        __syncwarp();
    } else if (TE && warp == 2) {
        if (elect_one()) {
            // ---------------- C store issuer: slot -> global (fp32 + 16-bit image), recycle
            constexpr int kChunks = BN / 32;
            int cnt = 0, prev = -1;
            for (int u = ubeg; u < args.units; u += ustep, ++cnt) {
                int t0, tj, z, kb0, kb1;
                unit_coords<MODE>(args, u, t0, tj, z, kb0, kb1);
                for (int ch = 0; ch < kChunks; ++ch) {
                    int s;
                    uint32_t round;
                    te_slot<kChunks, EPI_WG, kNcw>(cnt, ch, s, round);
                    mbar_wait(&cready_bar[s], round & 1u);
                    if (args.c_ef)
                        tma_store_2d_hint(&tmC, epi_buf + s * (C::kCSlot / 4), t0, tj * BN + ch * 32,
                                          policy_evict_first());
                    else
                        tma_store_2d(&tmC, epi_buf + s * (C::kCSlot / 4), t0, tj * BN + ch * 32);
                    bulk_commit();
                    bulk_wait_read<1>();   // the previous chunk's slot has been read out: recycle it
                    if (prev >= 0) mbar_arrive(&cempty_bar[prev]);
                    prev = s;
                }
            }
            bulk_wait<0>();
        }
        __syncwarp();
    } else if (TE && warp >= 4) {
        // ---------------- TMA epilogue warps: ew = TMEM lane quarter (32 rows), wg = chunk interleave
        constexpr int kChunks = BN / 32;
        const int ew = warp & 3;
        const int wg = (warp - 4) >> 2;
        const uint32_t lane_off = static_cast<uint32_t>(ew * 32) << 16;
        const bool hv = args.Ch != nullptr;
        int cnt = 0;
        for (int u = ubeg; u < args.units; u += ustep, ++cnt) {
            int t0, tj, z, kb0, kb1;
            unit_coords<MODE>(args, u, t0, tj, z, kb0, kb1);
            const int64_t row = (int64_t)t0 + ew * 32 + lane;
            const int acc = cnt % C::kAcc;
            const uint32_t aphase = (uint32_t)(cnt / C::kAcc) & 1u;
            bool waited = false;
            for (int ch = wg; ch < kChunks; ch += EPI_WG) {
                int s;
                uint32_t round;
                te_slot<kChunks, EPI_WG, kNcw>(cnt, ch, s, round);
                if (!waited) {
                    mbar_wait(&tfull_bar[acc], aphase);
                    tc_fence_after();
                    waited = true;
                }
                uint32_t v[32];
                tmem_ld32(tmem_base + acc * C::kAccCols + lane_off + ch * 32, v);
                tmem_ld_wait();
                if (ch + EPI_WG >= kChunks) {
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&tempty_bar[acc]);
                }
                mbar_wait(&cfull_bar[s], round & 1u);
                float* cs = epi_buf + s * (C::kCSlot / 4) + ew * 32 + lane;   // [col][128 rows]
                const int j0 = tj * BN + ch * 32;
                uint16_t* hp = hv ? reinterpret_cast<uint16_t*>(args.Ch) + row + (int64_t)j0 * args.ldh : nullptr;
                const int jmax = (row < args.m && j0 + 32 > args.h0) ? min(32, args.w - j0) : 0;
                const int jmin = args.h0 - j0;
#pragma unroll
                for (int jj = 0; jj < 32; ++jj) {
                    const float d = __uint_as_float(v[jj]);
                    const float x = args.overwrite ? d : cs[jj * kBM] - d;
                    cs[jj * kBM] = x;
                    if (hv && jj < jmax && jj >= jmin) hp[(int64_t)jj * args.ldh] = f2h_bits(x, args.bf16);
                }
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) mbar_arrive(&cready_bar[s]);
            }
            if (!waited) {
                mbar_wait(&tfull_bar[acc], aphase);
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&tempty_bar[acc]);
            }
        }
    } else if (!TE && warp >= 4) {
        // ---------------- epilogue warps: ew = TMEM lane quarter, wg = column interleave
        const int ew = warp & 3;
        const int wg = (warp - 4) >> 2;
        float* tb = epi_buf + (warp - 4) * 32 * kEpiLd;
        const uint32_t lane_off = static_cast<uint32_t>(ew * 32) << 16;
        const int q = lane & 7;       // row quad within the warp's 32 rows
        const int jsub = lane >> 3;   // column within a group of 4
        int cnt = 0;
        constexpr int kChunks = BN / 32;
        const bool rmw = (MODE == 1) && !args.overwrite;
        // measured: the one-chunk-ahead prefetch pays off at BN = 256 (4-8 chunks per tile) and
        // costs a little at the narrow levels, which keep the per-chunk load
        constexpr bool kAhead = (BN >= 256);
        // K2: the fp32 C values of a chunk are loaded one chunk ahead (the next tile's first
        // chunk during the current tile's last), so each epilogue warp keeps two chunks of
        // HBM reads in flight instead of paying a full memory latency per chunk.
        auto load_old = [&](int t0x, int t1x, int chx, float4 (&o)[8]) {
            const int64_t r0x = (int64_t)t0x + ew * 32 + 4 * q;
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                const int j = t1x + chx * 32 + k * 4 + jsub;
                const float* cp = args.C + r0x + (int64_t)j * args.ldc;
                if (j < args.w && r0x + 3 < args.m && args.vec_ok) {
                    o[k] = __ldcs(reinterpret_cast<const float4*>(cp));
                } else {
                    o[k].x = (j < args.w && r0x + 0 < args.m) ? cp[0] : 0.f;
                    o[k].y = (j < args.w && r0x + 1 < args.m) ? cp[1] : 0.f;
                    o[k].z = (j < args.w && r0x + 2 < args.m) ? cp[2] : 0.f;
                    o[k].w = (j < args.w && r0x + 3 < args.m) ? cp[3] : 0.f;
                }
            }
        };
        float4 old[8], nxt[8];
        if (kAhead && rmw && ubeg < args.units && wg < kChunks) {
            int t0, tj, z, kb0, kb1;
            unit_coords<MODE>(args, ubeg, t0, tj, z, kb0, kb1);
            load_old(t0, tj * BN, wg, old);
        }
        for (int u = ubeg; u < args.units; u += ustep, ++cnt) {
            int t0, tj, z, kb0, kb1;
            unit_coords<MODE>(args, u, t0, tj, z, kb0, kb1);
            const int t1 = tj * BN;
            const int acc = cnt % C::kAcc;
            const uint32_t aphase = (uint32_t)(cnt / C::kAcc) & 1u;
            const int64_t row0 = (int64_t)t0 + ew * 32 + 4 * q;   // first of this lane's 4 rows
            bool waited = false;
            for (int ch = wg; ch < kChunks; ch += EPI_WG) {
                const int c = ch * 32;
                if (!kAhead && rmw) load_old(t0, t1, ch, old);
                if (kAhead && rmw) {
                    if (ch + EPI_WG < kChunks) {
                        load_old(t0, t1, ch + EPI_WG, nxt);
                    } else if (u + ustep < args.units) {
                        int t0n, tjn, zn, kb0n, kb1n;
                        unit_coords<MODE>(args, u + ustep, t0n, tjn, zn, kb0n, kb1n);
                        load_old(t0n, tjn * BN, wg, nxt);
                    }
                }
                if (!waited) {
                    mbar_wait(&tfull_bar[acc], aphase);
                    tc_fence_after();
                    waited = true;
                }
                const uint32_t dtm = tmem_base + acc * C::kAccCols + lane_off;
                uint32_t v[32];
                tmem_ld32(dtm + c, v);
                tmem_ld_wait();
                float d[32];
#pragma unroll
                for (int jj = 0; jj < 32; ++jj) d[jj] = __uint_as_float(v[jj]);
                if (SPLIT) {
                    tmem_ld32(dtm + BN + c, v);
                    tmem_ld_wait();
#pragma unroll
                    for (int jj = 0; jj < 32; ++jj) d[jj] += __uint_as_float(v[jj]) * (1.0f / 2048.0f);
                }
                if (ch + EPI_WG >= kChunks) {
                    // last TMEM read of this accumulator by this warp: release it early
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&tempty_bar[acc]);
                }
                // ---- transpose through smem: tb[j][row] (row = lane)
#pragma unroll
                for (int jj = 0; jj < 32; ++jj) tb[jj * kEpiLd + lane] = d[jj];
                __syncwarp();
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    const int jl = k * 4 + jsub;
                    const int j = t1 + c + jl;
                    const float4 dv = *reinterpret_cast<const float4*>(tb + jl * kEpiLd + 4 * q);
                    if (MODE == 0) {
                        // the partial buffer is padded to whole tiles: always in range, 16B aligned
                        float* out = args.P + (int64_t)z * args.p_stride + (int64_t)j * args.ldp + row0;
                        *reinterpret_cast<float4*>(out) = dv;
                    } else if (j < args.w) {
                        float4 nv;
                        if (args.overwrite) {
                            nv = dv;
                        } else {
                            nv.x = old[k].x - dv.x;
                            nv.y = old[k].y - dv.y;
                            nv.z = old[k].z - dv.z;
                            nv.w = old[k].w - dv.w;
                        }
                        float* cp = args.C + row0 + (int64_t)j * args.ldc;
                        uint16_t* hp = (args.Ch && j >= args.h0) ? reinterpret_cast<uint16_t*>(args.Ch) + row0 + (int64_t)j * args.ldh
                                               : nullptr;
                        uint16_t* lp = args.Cl ? reinterpret_cast<uint16_t*>(args.Cl) + row0 + (int64_t)j * args.ldh
                                               : nullptr;
                        const float nvv[4] = {nv.x, nv.y, nv.z, nv.w};
                        ushort4 hb, lb;
                        uint16_t* hbp = reinterpret_cast<uint16_t*>(&hb);
                        uint16_t* lbp = reinterpret_cast<uint16_t*>(&lb);
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            hbp[e] = f2h_bits(nvv[e], args.bf16);
                            lbp[e] = f2h_bits((nvv[e] - h2f_bits(hbp[e], args.bf16)) * 2048.0f, args.bf16);
                        }
                        if (row0 + 3 < args.m && args.vec_ok) {
                            __stcs(reinterpret_cast<float4*>(cp), nv);
                            if (hp) *reinterpret_cast<ushort4*>(hp) = hb;
                            if (lp) *reinterpret_cast<ushort4*>(lp) = lb;
                        } else {
#pragma unroll
                            for (int e = 0; e < 4; ++e)
                                if (row0 + e < args.m) {
                                    cp[e] = nvv[e];
                                    if (hp) hp[e] = hbp[e];
                                    if (lp) lp[e] = lbp[e];
                                }
                        }
                    }
                }
                __syncwarp();
                if (kAhead && rmw) {
#pragma unroll
                    for (int k = 0; k < 8; ++k) old[k] = nxt[k];
                }
            }
            if (!waited) {   // this warp had no chunk (EPI_WG > chunks): still consume the phase
                mbar_wait(&tfull_bar[acc], aphase);
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&tempty_bar[acc]);
            }
        }
    }

    tc_fence_before();
    __syncthreads();
    if (args.mc) cluster_sync_all();   // no CTA exits while its peer may still signal its barriers
    if (warp == 2) tmem_dealloc<C::kTmemCols>(tmem_base);
}

// --------------------------------------------------------------------------------------
// split-K reduction for K1: R12(i,j) = sum_z P[z](i,j) in fixed z order (deterministic),
// written as fp32 into R (ldr) and rounded to 16 bit (hi, and lo for split mode) into
// the K2 B-operand image R12h (K-major: column j holds R12(:, j), ld = ldh).
template <int LANES>
__global__ void __launch_bounds__(32 * LANES) proj_reduce_kernel(const float* __restrict__ P, int64_t ldp,
                                                                int64_t p_stride, int splits, int h, int w,
                                                                float* __restrict__ R, int64_t ldr,
                                                                float* __restrict__ Rf, int64_t ldf,
                                                                uint16_t* __restrict__ Rh, uint16_t* __restrict__ Rl,
                                                                int64_t ldh, int bf16) {
    RG_PDL_ENTRY();
    // block (32, LANES): 32 consecutive outputs x LANES split lanes; lane ty sums splits
    // ty, ty+LANES, ... in order, then the lane sums are added in order (deterministic).
    __shared__ float part[LANES][33];
    const int64_t total = (int64_t)h * w;
    const int64_t e = (int64_t)blockIdx.x * 32 + threadIdx.x;
    const bool valid = e < total;
    const int i = valid ? (int)(e % h) : 0;
    const int j = valid ? (int)(e / h) : 0;
    const float* p = P + (int64_t)j * ldp + i;
    float s = 0.f;
    if (valid) {
        int z = threadIdx.y;
        for (; z + 3 * LANES < splits; z += 4 * LANES) {
            const float a = __ldcg(p + (int64_t)z * p_stride), b = __ldcg(p + (int64_t)(z + LANES) * p_stride);
            const float c = __ldcg(p + (int64_t)(z + 2 * LANES) * p_stride);
            const float d = __ldcg(p + (int64_t)(z + 3 * LANES) * p_stride);
            s += a; s += b; s += c; s += d;
        }
        for (; z < splits; z += LANES) s += __ldcg(p + (int64_t)z * p_stride);
    }
    part[threadIdx.y][threadIdx.x] = s;
    __syncthreads();
    if (threadIdx.y != 0 || !valid) return;
    float t = 0.f;
#pragma unroll
    for (int y = 0; y < LANES; ++y) t += part[y][threadIdx.x];
    if (R) R[i + (int64_t)j * ldr] = t;
    if (Rf) Rf[i + (int64_t)j * ldf] = t;
    if (Rh) {
        const uint16_t hb = f2h_bits(t, bf16);
        Rh[i + (int64_t)j * ldh] = hb;
        if (Rl) Rl[i + (int64_t)j * ldh] = f2h_bits((t - h2f_bits(hb, bf16)) * 2048.0f, bf16);
    }
}

// Same reduction for large outputs: persistent grid-stride blocks, each unit = 128 consecutive
// rows i (4 per lane, float4 loads; the partial buffers are padded to whole 128-row tiles) of
// one column j, LANES split lanes.  The one-output-per-thread kernel above spends most of its
// time scheduling ~10^5 tiny blocks at the top recursion levels.
template <int LANES>
__global__ void __launch_bounds__(32 * LANES) proj_reduce4_kernel(const float* __restrict__ P, int64_t ldp,
                                                                 int64_t p_stride, int splits, int h, int w,
                                                                 float* __restrict__ R, int64_t ldr,
                                                                 float* __restrict__ Rf, int64_t ldf,
                                                                 uint16_t* __restrict__ Rh, uint16_t* __restrict__ Rl,
                                                                 int64_t ldh, int bf16) {
    RG_PDL_ENTRY();
    __shared__ float4 part[LANES][33];
    const int nic = (h + 127) / 128;
    const int units = nic * w;
    const int tx = threadIdx.x, ty = threadIdx.y;
    for (int u = blockIdx.x; u < units; u += gridDim.x) {
        const int ic = u % nic, j = u / nic;
        const int i0 = ic * 128 + 4 * tx;
        const float* p = P + (int64_t)j * ldp + i0;
        float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
        int z = ty;
        for (; z + 3 * LANES < splits; z += 4 * LANES) {
            const float4 a = __ldcg(reinterpret_cast<const float4*>(p + (int64_t)z * p_stride));
            const float4 b = __ldcg(reinterpret_cast<const float4*>(p + (int64_t)(z + LANES) * p_stride));
            const float4 c = __ldcg(reinterpret_cast<const float4*>(p + (int64_t)(z + 2 * LANES) * p_stride));
            const float4 d = __ldcg(reinterpret_cast<const float4*>(p + (int64_t)(z + 3 * LANES) * p_stride));
            s.x += a.x; s.y += a.y; s.z += a.z; s.w += a.w;
            s.x += b.x; s.y += b.y; s.z += b.z; s.w += b.w;
            s.x += c.x; s.y += c.y; s.z += c.z; s.w += c.w;
            s.x += d.x; s.y += d.y; s.z += d.z; s.w += d.w;
        }
        for (; z < splits; z += LANES) {
            const float4 a = __ldcg(reinterpret_cast<const float4*>(p + (int64_t)z * p_stride));
            s.x += a.x; s.y += a.y; s.z += a.z; s.w += a.w;
        }
        part[ty][tx] = s;
        __syncthreads();
        if (ty == 0) {
            float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
            for (int y = 0; y < LANES; ++y) {
                const float4 v = part[y][tx];
                t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
            }
            const float tv[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                const int i = i0 + e;
                if (i < h) {
                    if (R) R[i + (int64_t)j * ldr] = tv[e];
                    if (Rf) Rf[i + (int64_t)j * ldf] = tv[e];
                    if (Rh) {
                        const uint16_t hb = f2h_bits(tv[e], bf16);
                        Rh[i + (int64_t)j * ldh] = hb;
                        if (Rl) Rl[i + (int64_t)j * ldh] = f2h_bits((tv[e] - h2f_bits(hb, bf16)) * 2048.0f, bf16);
                    }
                }
            }
        }
        __syncthreads();
    }
}

// Few splits (the wide levels, where the tile count already fills the machine): a plain
// grid-stride pass, 4 consecutive rows i per thread (float4, the partial buffers are padded to
// whole 128-row tiles), all splits summed in order z = 0, 1, ... by that thread (deterministic).
// The split-lane kernel above leaves most lanes idle here and pays two block barriers per
// 128-row unit.
__global__ void __launch_bounds__(256) proj_reduce_few_kernel(const float* __restrict__ P, int64_t ldp,
                                                              int64_t p_stride, int splits, int h, int w,
                                                              float* __restrict__ R, int64_t ldr,
                                                              float* __restrict__ Rf, int64_t ldf,
                                                              uint16_t* __restrict__ Rh, uint16_t* __restrict__ Rl,
                                                              int64_t ldh, int bf16) {
    RG_PDL_ENTRY();
    const int h4 = (h + 3) >> 2;
    const int64_t groups = (int64_t)h4 * w;
    for (int64_t gi = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; gi < groups;
         gi += (int64_t)gridDim.x * blockDim.x) {
        const int i0 = 4 * (int)(gi % h4), j = (int)(gi / h4);
        const float* p = P + (int64_t)j * ldp + i0;
        float4 v[8];
#pragma unroll
        for (int z = 0; z < 8; ++z)
            if (z < splits) v[z] = __ldcg(reinterpret_cast<const float4*>(p + (int64_t)z * p_stride));
        float4 t = v[0];
#pragma unroll
        for (int z = 1; z < 8; ++z)
            if (z < splits) {
                t.x += v[z].x; t.y += v[z].y; t.z += v[z].z; t.w += v[z].w;
            }
        const float tv[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
        for (int e = 0; e < 4; ++e) {
            const int i = i0 + e;
            if (i < h) {
                if (R) R[i + (int64_t)j * ldr] = tv[e];
                if (Rf) Rf[i + (int64_t)j * ldf] = tv[e];
                if (Rh) {
                    const uint16_t hb = f2h_bits(tv[e], bf16);
                    Rh[i + (int64_t)j * ldh] = hb;
                    if (Rl) Rl[i + (int64_t)j * ldh] = f2h_bits((tv[e] - h2f_bits(hb, bf16)) * 2048.0f, bf16);
                }
            }
        }
    }
}

// After a cross-rank allreduce of Rf: write R and the 16-bit images.
__global__ void proj_finish_kernel(const float* __restrict__ Rf, int64_t ldf, int h, int w, float* __restrict__ R,
                                   int64_t ldr, uint16_t* __restrict__ Rh, uint16_t* __restrict__ Rl, int64_t ldh,
                                   int bf16) {
    RG_PDL_ENTRY();
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
static int num_sms() { return dev_sms(); }

template <int MODE, int BN, int STAGES, bool SPLIT, int EPI_WG, int TE = 0>
static cudaError_t launch_gemm(int units, const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& al,
                               const CUtensorMap& bl, const GemmArgs& args, cudaStream_t st,
                               const CUtensorMap* mc = nullptr) {
    using C = GemmCfg<BN, STAGES, SPLIT, EPI_WG, TE>;
    static_assert(C::kTotal <= 227 * 1024, "shared memory budget");
    auto kern = gemm_tc_kernel<MODE, BN, STAGES, SPLIT, EPI_WG, TE>;
    {
        cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(kern), C::kTotal);
        if (e != cudaSuccess) return e;
    }
    // persistent grid: one CTA per SM (two when the footprint allows), never more than units
    const int per_sm = (C::kTotal <= 113 * 1024 && C::kTmemCols <= 256) ? 2 : 1;
    int grid = num_sms() * per_sm;
    if (grid > units) grid = units;
    RG_LAUNCH((kern), grid, C::kThreads, C::kTotal, st, a, b, al, bl, mc ? *mc : a, args);
    return cudaGetLastError();
}

// K2 on cluster pairs (args.mc): the two CTAs of a cluster take vertically adjacent 128-row tiles
// with the same B tile, each loads one half of B (bh: box 64 k x BN / 2 rows) and multicasts it to
// both, so the B operand -- the L2 traffic that bounds the wide top-level K2 (each R12 tile is
// re-read for every row tile) -- is fetched once per pair.  Persistent grid of pairs.
template <int MODE, int BN, int STAGES, bool SPLIT, int EPI_WG, int TE = 0>
static cudaError_t launch_gemm_pair(int units, const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& bh,
                                    const GemmArgs& args, cudaStream_t st, const CUtensorMap* mc) {
    using C = GemmCfg<BN, STAGES, SPLIT, EPI_WG, TE>;
    auto kern = gemm_tc_kernel<MODE, BN, STAGES, SPLIT, EPI_WG, TE>;
    {
        cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(kern), C::kTotal);
        if (e != cudaSuccess) return e;
    }
    int grid = num_sms() & ~1;
    if (grid > 2 * units) grid = 2 * units;
    ++g_launches;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(C::kThreads);
    cfg.dynamicSmemBytes = C::kTotal;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, a, b, a, bh, mc ? *mc : a, args);
    return e != cudaSuccess ? e : cudaGetLastError();
}

// K2 with the TMA epilogue.  Shared memory (<= 227 KB) is split between the operand ring and
// the C-chunk ring (16 KB per slot): the HBM-bound levels (few k-blocks per tile) trade operand
// stages for C chunks in flight, the tensor-bound top level (K = 2048) keeps three stages.
static cudaError_t dispatch_bn_te(int bn, int units, const CUtensorMap& a, const CUtensorMap& b, const GemmArgs& args,
                                  cudaStream_t st, const CUtensorMap* mc, const CUtensorMap* bh) {
    static const int deep_kb = getenv("RGSQR_K2_DEEP_KB") ? atoi(getenv("RGSQR_K2_DEEP_KB")) : 8;
    const bool pair_off = getenv("RGSQR_K2_PAIR") && getenv("RGSQR_K2_PAIR")[0] == '0';   // read per plan (tests toggle it)
    const bool deep = args.kb_h <= deep_kb;
    static const int pair_min_kb = getenv("RGSQR_K2_PAIR_KB") ? atoi(getenv("RGSQR_K2_PAIR_KB")) : 9;
    if (bn == 256 && args.kb_h >= pair_min_kb && bh && !pair_off && args.tiles_i % 2 == 0) {
        GemmArgs pa = args;
        pa.mc = 1;
        pa.units = (args.tiles_i / 2) * args.tiles_j;
        if (deep) return launch_gemm_pair<1, 256, 2, false, 2, 8>(pa.units, a, b, *bh, pa, st, mc);
        return launch_gemm_pair<1, 256, 3, false, 2, 4>(pa.units, a, b, *bh, pa, st, mc);
    }
    switch (bn) {
        case 32: return launch_gemm<1, 32, 3, false, 2, 8>(units, a, b, a, b, args, st, mc);
        case 64: return launch_gemm<1, 64, 2, false, 2, 10>(units, a, b, a, b, args, st, mc);
        case 128: return launch_gemm<1, 128, 2, false, 2, 10>(units, a, b, a, b, args, st, mc);
        case 256:
            if (deep) return launch_gemm<1, 256, 2, false, 2, 8>(units, a, b, a, b, args, st, mc);
            return launch_gemm<1, 256, 3, false, 2, 4>(units, a, b, a, b, args, st, mc);
        default: return cudaErrorInvalidValue;
    }
}

template <int MODE, bool SPLIT>
static cudaError_t dispatch_bn(int bn, int units, const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& al,
                               const CUtensorMap& bl, const GemmArgs& args, cudaStream_t st) {
    // stage counts keep smem <= 227 KB: stages * (16 KB + BN * 128 B) * ops + epilogue buffers
    switch (bn) {
        case 32: return launch_gemm<MODE, 32, 3, SPLIT, 2>(units, a, b, al, bl, args, st);
        case 64: return launch_gemm<MODE, 64, SPLIT ? 3 : 4, SPLIT, 2>(units, a, b, al, bl, args, st);
        case 128: return launch_gemm<MODE, 128, SPLIT ? 2 : 5, SPLIT, 2>(units, a, b, al, bl, args, st);
        case 256:
            // K2 at wide levels is bound by the fp32 read-modify-write of A2: 8 epilogue warps
            // (3 stages to fit) double the HBM traffic in flight; K1 keeps 4 stages
            if constexpr (MODE == 1 && !SPLIT) return launch_gemm<MODE, 256, 3, SPLIT, 2>(units, a, b, al, bl, args, st);
            else
            return launch_gemm<MODE, 256, SPLIT ? 2 : 4, SPLIT, 1>(units, a, b, al, bl, args, st);
        case 192:   // general GEMMs with N = 3 x 176 .. 3 x 192 (lowrank l = 528): 3 tiles instead of 2 full + 1 nearly empty
            if constexpr (MODE == 1 && !SPLIT) return launch_gemm<MODE, 192, 4, SPLIT, 2>(units, a, b, al, bl, args, st);
            else
            return launch_gemm<MODE, 192, SPLIT ? 2 : 4, SPLIT, 1>(units, a, b, al, bl, args, st);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_proj_gemm(int bn, bool split, int tiles_i, int tiles_j, int splits, const CUtensorMap& q1,
                             const CUtensorMap& a2, const CUtensorMap& q1_lo, const CUtensorMap& a2_lo, float* P,
                             int64_t ldp, int64_t p_stride, int kb_total, int kb_per_split, int bf16,
                             cudaStream_t st, int jfast) {
    GemmArgs args{};
    args.jfast = jfast;
    args.units = tiles_i * tiles_j * splits;
    args.tiles_i = tiles_i;
    args.tiles_j = tiles_j;
    args.P = P;
    args.ldp = ldp;
    args.p_stride = p_stride;
    args.kb_total = kb_total;
    args.kb_per_split = kb_per_split;
    args.bf16 = bf16;
    args.vec_ok = 1;
    return split ? dispatch_bn<0, true>(bn, args.units, q1, a2, q1_lo, a2_lo, args, st)
                 : dispatch_bn<0, false>(bn, args.units, q1, a2, q1, a2, args, st);
}

cudaError_t launch_update_gemm(int bn, bool split, int64_t m, int w, int h, const CUtensorMap& q1_mn,
                               const CUtensorMap& r12, const CUtensorMap& q1_mn_lo, const CUtensorMap& r12_lo,
                               float* C, int64_t ldc, void* Ch, void* Cl, int64_t ldh, int bf16, cudaStream_t st,
                               int overwrite, const CUtensorMap* mc, int h0) {
    GemmArgs args{};
    args.overwrite = overwrite;
    args.h0 = h0;
    static const bool c_ef = !getenv("RGSQR_K2_NO_EF");
    args.c_ef = c_ef ? 1 : 0;
    args.C = C;
    args.ldc = ldc;
    args.Ch = Ch;
    args.Cl = Cl;
    args.ldh = ldh;
    args.m = m;
    args.w = w;
    args.kb_h = (h + kBK - 1) / kBK;
    args.bf16 = bf16;
    args.tiles_i = (int)((m + kBM - 1) / kBM);
    args.tiles_j = (w + bn - 1) / bn;
    args.units = args.tiles_i * args.tiles_j;
    args.vec_ok = ((ldc & 3) == 0) && ((reinterpret_cast<uintptr_t>(C) & 15) == 0) && ((ldh & 3) == 0) &&
                  ((reinterpret_cast<uintptr_t>(Ch) & 7) == 0) && ((reinterpret_cast<uintptr_t>(Cl) & 7) == 0);
    if (!split && mc && !Cl && !getenv("RGSQR_NO_TMA_EPI"))
        return dispatch_bn_te(bn, args.units, q1_mn, r12, args, st, mc, &r12_lo);
    return split ? dispatch_bn<1, true>(bn, args.units, q1_mn, r12, q1_mn_lo, r12_lo, args, st)
                 : dispatch_bn<1, false>(bn, args.units, q1_mn, r12, q1_mn, r12, args, st);
}

cudaError_t launch_proj_reduce(const float* P, int64_t ldp, int64_t p_stride, int splits, int h, int w, float* R,
                               int64_t ldr, float* Rf, int64_t ldf, uint16_t* Rh, uint16_t* Rl, int64_t ldh, int bf16,
                               cudaStream_t st) {
    const int64_t total = (int64_t)h * w;
    const bool aligned = (ldp & 3) == 0 && (p_stride & 3) == 0 && (reinterpret_cast<uintptr_t>(P) & 15) == 0;
    const int64_t units = (int64_t)((h + 127) / 128) * w;
    if (aligned && splits <= 8) {
        const int64_t groups = (int64_t)((h + 3) / 4) * w;
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((groups + 255) / 256, (int64_t)num_sms() * 8));
        RG_LAUNCH((proj_reduce_few_kernel), grid, 256, 0, st, P, ldp, p_stride, splits, h, w, R, ldr, Rf, ldf, Rh, Rl,
                  ldh, bf16);
    } else if (aligned && splits > 32 && units <= (int64_t)num_sms() * 2) {
        // narrow levels (many splits, few outputs): one wave of 1024-thread CTAs, 128 x 1 outputs per
        // CTA, every split lane's float4 loads in flight at once
        RG_LAUNCH((proj_reduce4_kernel<32>), (unsigned)units, dim3(32, 32), 0, st, P, ldp, p_stride, splits, h, w, R,
                  ldr, Rf, ldf, Rh, Rl, ldh, bf16);
    } else if (total >= 65536 && aligned) {
        const int grid = (int)std::min<int64_t>(units, (int64_t)num_sms() * 8);
        RG_LAUNCH((proj_reduce4_kernel<8>), grid, dim3(32, 8), 0, st, P, ldp, p_stride, splits, h, w, R, ldr, Rf, ldf,
                  Rh, Rl, ldh, bf16);
    } else if (splits > 32)
        RG_LAUNCH((proj_reduce_kernel<32>), (unsigned)((total + 31) / 32), dim3(32, 32), 0, st, P, ldp, p_stride, splits, h, w,
                                                                                       R, ldr, Rf, ldf, Rh, Rl, ldh,
                                                                                       bf16);
    else
        RG_LAUNCH((proj_reduce_kernel<8>), (unsigned)((total + 31) / 32), dim3(32, 8), 0, st, P, ldp, p_stride, splits, h, w, R,
                                                                                     ldr, Rf, ldf, Rh, Rl, ldh, bf16);
    return cudaGetLastError();
}

cudaError_t launch_proj_finish(const float* Rf, int64_t ldf, int h, int w, float* R, int64_t ldr, uint16_t* Rh,
                               uint16_t* Rl, int64_t ldh, int bf16, cudaStream_t st) {
    const int64_t total = (int64_t)h * w;
    int blocks = (int)((total + 255) / 256);
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    RG_LAUNCH((proj_finish_kernel), blocks, 256, 0, st, Rf, ldf, h, w, R, ldr, Rh, Rl, ldh, bf16);
    return cudaGetLastError();
}

}  // namespace rg
