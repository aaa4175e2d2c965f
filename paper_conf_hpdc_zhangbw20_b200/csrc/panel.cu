// panel.cu -- the leaf panelQR of Algorithm 1: the CAQR/TSQR panel of eq 8 (PAPER.md
// P:L221-237) built on fp32 modified Gram-Schmidt tiles (Algorithm 2).
//
//  (1) rows are split into balanced tiles of <= 256 rows; each CTA factors its tile with
//      MGS entirely in registers/shared memory (one HBM read of the panel);
//  (2)+(3) the tile R factors are stacked and factored by MGS again, 8 at a time, up a
//      tree; the last CTA to finish a group does the group's MGS ("last block" pattern:
//      __threadfence + atomic counter), so the whole tree runs inside the tile kernel;
//  (4)+(5) an apply kernel multiplies every tile Q by the product of its tree factors
//      and writes Q in fp32 plus the 16-bit shadow the tensor-core GEMMs read.
//
// Layout inside a CTA (256 threads, 8 warps): warp w owns panel columns w, w+8, w+16, w+24;
// lane l holds rows l, l+32, ..., l+224 of those columns, so a column norm or dot product
// is a per-lane partial sum + a 5-step warp shuffle, and the current q_k is broadcast
// through a double-buffered shared vector (one __syncthreads per MGS step).
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>

#include "kernels.h"

namespace rg {

constexpr int PNB = 32;    // panel width ("we fix our panel to be of 32 columns")
constexpr int PT = 256;    // max rows per tile
constexpr int PRPL = PT / 32;
constexpr int PG = 8;      // tree fan-in: 8 stacked 32x32 R's = 256 rows

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__device__ __forceinline__ uint16_t to16(float x, int bf16) {
    if (bf16) {
        __nv_bfloat16 b = __float2bfloat16_rn(x);
        return *reinterpret_cast<uint16_t*>(&b);
    }
    __half h = __float2half_rn(x);
    return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float from16(uint16_t u, int bf16) {
    if (bf16) return __bfloat162float(*reinterpret_cast<__nv_bfloat16*>(&u));
    return __half2float(*reinterpret_cast<__half*>(&u));
}

// MGS (Alg 2) on a <= 256 x nc tile held as a[t][i] = X(lane + 32 i, warp + 8 t).
// Rs (32 x 33 smem, zeroed by the caller) receives R; qbuf is 2 x 256 floats of smem.
// Returns (in *bad, smem) the first column with a zero / non-finite norm, or -1.
__device__ void mgs_tile(float (&a)[4][PRPL], int nc, float* qbuf, float (*Rs)[33], int* bad) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int k = 0; k < nc; ++k) {
        const int ow = k & 7, ot = k >> 3;
        float* qb = qbuf + (k & 1) * PT;
        if (warp == ow) {
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                if (t == ot) {
                    float s = 0.f;
#pragma unroll
                    for (int i = 0; i < PRPL; ++i) s = fmaf(a[t][i], a[t][i], s);
                    s = warp_sum(s);
                    const float rkk = sqrtf(s);                       // line 5
                    const bool ok = rkk > 0.f && isfinite(rkk);
#pragma unroll
                    for (int i = 0; i < PRPL; ++i) {
                        a[t][i] = ok ? __fdiv_rn(a[t][i], rkk) : 0.f;  // line 6
                        qb[lane + 32 * i] = a[t][i];
                    }
                    if (lane == 0) {
                        Rs[k][k] = ok ? rkk : 0.f;
                        if (!ok) atomicMin(bad, k);
                    }
                }
            }
        }
        __syncthreads();
        float q[PRPL];
#pragma unroll
        for (int i = 0; i < PRPL; ++i) q[i] = qb[lane + 32 * i];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const int c = warp + 8 * t;
            if (c > k && c < nc) {
                float d = 0.f;
#pragma unroll
                for (int i = 0; i < PRPL; ++i) d = fmaf(q[i], a[t][i], d);
                d = warp_sum(d);                                      // line 7
#pragma unroll
                for (int i = 0; i < PRPL; ++i) a[t][i] = fmaf(-d, q[i], a[t][i]);  // line 8
                if (lane == 0) Rs[k][c] = d;
            }
        }
    }
    __syncthreads();
}

struct PanelArgs {
    float* Q;          // panel columns (fp32, in/out, in place), ldq
    int64_t ldq;
    uint16_t* Qh;      // 16-bit shadow of the panel columns (hi), ldh
    uint16_t* Ql;      // lo part (split mode) or null
    int64_t ldh;
    int64_t m;
    int nc;            // columns in this panel (<= 32)
    int ntiles;
    int64_t base_rows, extra;   // tile t has base_rows + (t < extra) rows
    float* R;          // final nc x nc R block (ldr) -- or local R when distributed
    int64_t ldr;
    float* ws;         // tree workspace: R stacks and Q factors, 32x32 blocks
    int* counters;     // per tree node
    int levels;        // number of stacked levels above the tiles (0 if ntiles == 1)
    int lvl_n[8];      // N_L blocks at level L (lvl_n[0] = ntiles)
    int64_t r_off[8];  // ws offset (floats) of level-L R stack
    int64_t q_off[8];  // ws offset of level-L Q factors (L >= 1; indexed by child)
    int c_off[8];      // counter offset of level L groups
    int finalize;      // 1: single tile and not distributed -> write final Q/shadow/R directly
    int bf16;
    int col0;          // global index of the panel's first column (status reporting)
    int* status;       // [0] = first breakdown column (INT_MAX if none)
    const int* guard;  // non-null: run only if *guard != 0 (fallback of the CholQR2 panel)
};

__device__ __forceinline__ int64_t tile_row0(const PanelArgs& p, int t) {
    return (int64_t)t * p.base_rows + (t < p.extra ? t : p.extra);
}

__global__ void __launch_bounds__(256, 2) panel_tile_kernel(PanelArgs p) {
    RG_PDL_ENTRY();
    if (p.guard && *p.guard == 0) return;
    __shared__ float qbuf[2 * PT];
    __shared__ float Rs[PNB][33];
    __shared__ int bad;
    __shared__ int s_last;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int e = threadIdx.x; e < PNB * 33; e += blockDim.x) (&Rs[0][0])[e] = 0.f;
    if (threadIdx.x == 0) bad = 0x7fffffff;

    const int t = blockIdx.x;
    const int64_t r0 = tile_row0(p, t);
    const int rows = (int)(p.base_rows + (t < p.extra ? 1 : 0));
    float a[4][PRPL];
#pragma unroll
    for (int tt = 0; tt < 4; ++tt) {
        const int c = warp + 8 * tt;
#pragma unroll
        for (int i = 0; i < PRPL; ++i) {
            const int rr = lane + 32 * i;
            a[tt][i] = (c < p.nc && rr < rows) ? p.Q[r0 + rr + (int64_t)c * p.ldq] : 0.f;
        }
    }
    __syncthreads();
    mgs_tile(a, p.nc, qbuf, Rs, &bad);

    // tile Q -> global (final if single tile, else local factor overwritten by the apply pass)
#pragma unroll
    for (int tt = 0; tt < 4; ++tt) {
        const int c = warp + 8 * tt;
        if (c < p.nc) {
#pragma unroll
            for (int i = 0; i < PRPL; ++i) {
                const int rr = lane + 32 * i;
                if (rr < rows) {
                    const int64_t off = r0 + rr + (int64_t)c * p.ldq;
                    p.Q[off] = a[tt][i];
                    if (p.finalize && p.Qh) {
                        const int64_t hoff = r0 + rr + (int64_t)c * p.ldh;
                        const uint16_t hb = to16(a[tt][i], p.bf16);
                        p.Qh[hoff] = hb;
                        if (p.Ql) p.Ql[hoff] = to16((a[tt][i] - from16(hb, p.bf16)) * 2048.f, p.bf16);
                    }
                }
            }
        }
    }
    if (p.levels == 0) {
        // single tile: R is final (or the local R of a distributed panel)
        for (int e = threadIdx.x; e < p.nc * p.nc; e += blockDim.x) {
            const int i = e % p.nc, j = e / p.nc;
            p.R[i + (int64_t)j * p.ldr] = (i <= j) ? Rs[i][j] : 0.f;
        }
        if (threadIdx.x == 0 && bad != 0x7fffffff) atomicMin(p.status, p.col0 + bad);
        return;
    }
    // tile R -> level-0 stack
    float* R0 = p.ws + p.r_off[0] + (int64_t)t * PNB * PNB;
    for (int e = threadIdx.x; e < PNB * PNB; e += blockDim.x) {
        const int i = e & 31, j = e >> 5;
        R0[e] = (i <= j && j < p.nc) ? Rs[i][j] : 0.f;
    }
    if (threadIdx.x == 0 && bad != 0x7fffffff) atomicMin(p.status, p.col0 + bad);

    // climb the tree: the last CTA to arrive in a group factors the group's stacked R's
    int idx = t;
    for (int L = 1; L <= p.levels; ++L) {
        const int g = idx / PG;
        const int nchild = min(PG, p.lvl_n[L - 1] - g * PG);
        __threadfence();
        __syncthreads();
        if (threadIdx.x == 0) {
            const int old = atomicAdd(&p.counters[p.c_off[L] + g], 1);
            s_last = (old == nchild - 1);
        }
        __syncthreads();
        if (!s_last) return;
        __threadfence();
        if (threadIdx.x == 0) {
            p.counters[p.c_off[L] + g] = 0;   // every arrival for this node has happened
            bad = 0x7fffffff;
        }
        for (int e = threadIdx.x; e < PNB * 33; e += blockDim.x) (&Rs[0][0])[e] = 0.f;
        const float* Rst = p.ws + p.r_off[L - 1] + (int64_t)g * PG * PNB * PNB;
#pragma unroll
        for (int tt = 0; tt < 4; ++tt) {
            const int c = warp + 8 * tt;
#pragma unroll
            for (int i = 0; i < PRPL; ++i)   // stack row lane + 32 i = row `lane` of child block i
                a[tt][i] = (i < nchild) ? __ldcg(Rst + (int64_t)i * PNB * PNB + lane + 32 * c) : 0.f;
        }
        __syncthreads();
        mgs_tile(a, p.nc, qbuf, Rs, &bad);
        float* Qf = p.ws + p.q_off[L] + (int64_t)g * PG * PNB * PNB;
#pragma unroll
        for (int tt = 0; tt < 4; ++tt) {
            const int c = warp + 8 * tt;
#pragma unroll
            for (int i = 0; i < PRPL; ++i)
                if (i < nchild) Qf[(int64_t)i * PNB * PNB + lane + 32 * c] = a[tt][i];
        }
        if (threadIdx.x == 0 && bad != 0x7fffffff) atomicMin(p.status, p.col0 + bad);
        if (L == p.levels) {
            for (int e = threadIdx.x; e < p.nc * p.nc; e += blockDim.x) {
                const int i = e % p.nc, j = e / p.nc;
                p.R[i + (int64_t)j * p.ldr] = (i <= j) ? Rs[i][j] : 0.f;
            }
        } else {
            float* Rn = p.ws + p.r_off[L] + (int64_t)g * PNB * PNB;
            for (int e = threadIdx.x; e < PNB * PNB; e += blockDim.x) {
                const int i = e & 31, j = e >> 5;
                Rn[e] = (i <= j && j < p.nc) ? Rs[i][j] : 0.f;
            }
        }
        idx = g;
    }
}

// Step (4)+(5): Q_tile <- Q_tile * (Qf_1[t] * Qf_2[t/8] * ... * Gq), fp32 + 16-bit shadow.
// Gq (32x32, ld 32) is the rank's block of the cross-GPU stack factor, or null.
__global__ void __launch_bounds__(256) panel_apply_kernel(PanelArgs p, const float* __restrict__ Gq) {
    RG_PDL_ENTRY();
    if (p.guard && *p.guard == 0) return;
    __shared__ float M[PNB][PNB + 1];
    __shared__ float Tm[PNB][PNB + 1];
    __shared__ float F[PNB][PNB + 1];
    const int t = blockIdx.x;
    const int tid = threadIdx.x;
    // M = product of the tree factors along the tile's path, bottom-up
    if (p.levels >= 1) {
        const float* f = p.ws + p.q_off[1] + (int64_t)t * PNB * PNB;
        for (int e = tid; e < PNB * PNB; e += blockDim.x) M[e & 31][e >> 5] = __ldcg(f + e);
    } else {
        for (int e = tid; e < PNB * PNB; e += blockDim.x) M[e & 31][e >> 5] = ((e & 31) == (e >> 5)) ? 1.f : 0.f;
    }
    __syncthreads();
    int idx = t;
    for (int L = 2; L <= p.levels + 1; ++L) {
        const float* f;
        if (L <= p.levels) {
            idx /= PG;
            f = p.ws + p.q_off[L] + (int64_t)idx * PNB * PNB;
        } else {
            if (!Gq) break;
            f = Gq;
        }
        for (int e = tid; e < PNB * PNB; e += blockDim.x) F[e & 31][e >> 5] = __ldcg(f + e);
        __syncthreads();
        for (int e = tid; e < PNB * PNB; e += blockDim.x) {
            const int i = e & 31, j = e >> 5;
            float s = 0.f;
#pragma unroll 8
            for (int k = 0; k < PNB; ++k) s = fmaf(M[i][k], F[k][j], s);
            Tm[i][j] = s;
        }
        __syncthreads();
        for (int e = tid; e < PNB * PNB; e += blockDim.x) M[e & 31][e >> 5] = Tm[e & 31][e >> 5];
        __syncthreads();
    }
    if (p.levels == 0 && Gq) {  // single tile, distributed: M = Gq
        for (int e = tid; e < PNB * PNB; e += blockDim.x) M[e & 31][e >> 5] = __ldcg(Gq + e);
        __syncthreads();
    }
    const int64_t r0 = tile_row0(p, t);
    const int rows = (int)(p.base_rows + (t < p.extra ? 1 : 0));
    for (int rr = tid; rr < rows; rr += blockDim.x) {
        const int64_t row = r0 + rr;
        float q[PNB];
#pragma unroll
        for (int c = 0; c < PNB; ++c) q[c] = (c < p.nc) ? p.Q[row + (int64_t)c * p.ldq] : 0.f;
#pragma unroll 4
        for (int j = 0; j < p.nc; ++j) {
            float s = 0.f;
#pragma unroll
            for (int c = 0; c < PNB; ++c) s = fmaf(q[c], M[c][j], s);
            p.Q[row + (int64_t)j * p.ldq] = s;
            if (p.Qh) {
                const uint16_t hb = to16(s, p.bf16);
                p.Qh[row + (int64_t)j * p.ldh] = hb;
                if (p.Ql) p.Ql[row + (int64_t)j * p.ldh] = to16((s - from16(hb, p.bf16)) * 2048.f, p.bf16);
            }
        }
    }
}

// Cross-rank TSQR top (eq 8 at GPU granularity): the P local R's (P <= 8,
// gathered as P x (32x32) blocks) are stacked and factored by MGS; writes the final R
// and the P Q-blocks (each 32x32) of the stack factor.
__global__ void __launch_bounds__(256) panel_stack_kernel(const float* __restrict__ Rall, int P, int nc, float* R,
                                                          int64_t ldr, float* Qblocks, int* status, int col0,
                                                          const int* guard) {
    RG_PDL_ENTRY();
    if (guard && *guard == 0) return;
    __shared__ float qbuf[2 * PT];
    __shared__ float Rs[PNB][33];
    __shared__ int bad;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int e = threadIdx.x; e < PNB * 33; e += blockDim.x) (&Rs[0][0])[e] = 0.f;
    if (threadIdx.x == 0) bad = 0x7fffffff;
    float a[4][PRPL];
#pragma unroll
    for (int tt = 0; tt < 4; ++tt) {
        const int c = warp + 8 * tt;
#pragma unroll
        for (int i = 0; i < PRPL; ++i) {
            const int rr = lane;  // block i, row `lane` of the nc x nc local R (ld = nc)
            a[tt][i] = (i < P && c < nc && rr < nc) ? Rall[(int64_t)i * nc * nc + rr + (int64_t)c * nc] : 0.f;
        }
    }
    __syncthreads();
    mgs_tile(a, nc, qbuf, Rs, &bad);
#pragma unroll
    for (int tt = 0; tt < 4; ++tt) {
        const int c = warp + 8 * tt;
#pragma unroll
        for (int i = 0; i < PRPL; ++i)
            if (i < P) Qblocks[(int64_t)i * PNB * PNB + lane + 32 * c] = (c < nc && lane < nc) ? a[tt][i] : 0.f;
    }
    for (int e = threadIdx.x; e < nc * nc; e += blockDim.x) {
        const int i = e % nc, j = e / nc;
        R[i + (int64_t)j * ldr] = (i <= j) ? Rs[i][j] : 0.f;
    }
    if (threadIdx.x == 0 && bad != 0x7fffffff) atomicMin(status, col0 + bad);
}

// ------------------------------------------------------------------ host side
int panel_levels(int ntiles, int* lvl_n) {
    int L = 0;
    lvl_n[0] = ntiles;
    while (lvl_n[L] > 1) {
        lvl_n[L + 1] = (lvl_n[L] + PG - 1) / PG;
        ++L;
    }
    return L;
}

size_t panel_ws_floats(int64_t m) {
    const int ntiles = (int)((m + PT - 1) / PT);
    int lvl_n[16];
    const int L = panel_levels(ntiles, lvl_n);
    size_t f = 0;
    for (int l = 0; l <= L; ++l) f += (size_t)lvl_n[l] * PNB * PNB * 2;
    return f + 1024;
}

size_t panel_counters(int64_t m) {
    const int ntiles = (int)((m + PT - 1) / PT);
    int lvl_n[16];
    const int L = panel_levels(ntiles, lvl_n);
    size_t c = 0;
    for (int l = 0; l <= L; ++l) c += lvl_n[l];
    return c + 8;
}

cudaError_t launch_panel(const PanelLaunch& pl, cudaStream_t st) {
    PanelArgs p{};
    p.Q = pl.Q;
    p.ldq = pl.ldq;
    p.Qh = pl.Qh;
    p.Ql = pl.Ql;
    p.ldh = pl.ldh;
    p.m = pl.m;
    p.nc = pl.nc;
    p.ntiles = (int)((pl.m + PT - 1) / PT);
    if (p.ntiles < 1) p.ntiles = 1;
    p.base_rows = pl.m / p.ntiles;
    p.extra = pl.m % p.ntiles;
    p.ldr = pl.ldr;
    p.R = pl.R;
    p.ws = pl.ws;
    p.counters = pl.counters;
    int lvl_n[16];
    p.levels = panel_levels(p.ntiles, lvl_n);
    if (p.levels > 7) return cudaErrorInvalidValue;
    int64_t off = 0;
    int coff = 0;
    for (int l = 0; l <= p.levels; ++l) {
        p.lvl_n[l] = lvl_n[l];
        p.r_off[l] = off;
        off += (int64_t)lvl_n[l] * PNB * PNB;
        p.c_off[l] = coff;
        coff += lvl_n[l];
    }
    for (int l = 1; l <= p.levels; ++l) {
        p.q_off[l] = off;
        off += (int64_t)lvl_n[l - 1] * PNB * PNB;
    }
    p.finalize = (p.levels == 0 && !pl.distributed) ? 1 : 0;
    p.bf16 = pl.bf16;
    p.col0 = pl.col0;
    p.status = pl.status;
    p.guard = pl.guard;
    RG_LAUNCH((panel_tile_kernel), p.ntiles, 256, 0, st, p);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    if (pl.distributed) return cudaSuccess;  // caller gathers R, then calls launch_panel_apply
    if (p.levels > 0) {
        RG_LAUNCH((panel_apply_kernel), p.ntiles, 256, 0, st, p, nullptr);
        e = cudaGetLastError();
    }
    return e;
}

cudaError_t launch_panel_apply(const PanelLaunch& pl, const float* Gq, cudaStream_t st) {
    PanelArgs p{};
    p.Q = pl.Q;
    p.ldq = pl.ldq;
    p.Qh = pl.Qh;
    p.Ql = pl.Ql;
    p.ldh = pl.ldh;
    p.m = pl.m;
    p.nc = pl.nc;
    p.ntiles = (int)((pl.m + PT - 1) / PT);
    if (p.ntiles < 1) p.ntiles = 1;
    p.base_rows = pl.m / p.ntiles;
    p.extra = pl.m % p.ntiles;
    p.ws = pl.ws;
    int lvl_n[16];
    p.levels = panel_levels(p.ntiles, lvl_n);
    int64_t off = 0;
    for (int l = 0; l <= p.levels; ++l) off += (int64_t)lvl_n[l] * PNB * PNB;
    for (int l = 1; l <= p.levels; ++l) {
        p.q_off[l] = off;
        off += (int64_t)lvl_n[l - 1] * PNB * PNB;
    }
    p.bf16 = pl.bf16;
    p.guard = pl.guard;
    RG_LAUNCH((panel_apply_kernel), p.ntiles, 256, 0, st, p, Gq);
    return cudaGetLastError();
}

cudaError_t launch_panel_stack(const float* Rall, int P, int nc, float* R, int64_t ldr, float* Qblocks, int* status,
                               int col0, const int* guard, cudaStream_t st) {
    RG_LAUNCH((panel_stack_kernel), 1, 256, 0, st, Rall, P, nc, R, ldr, Qblocks, status, col0, guard);
    return cudaGetLastError();
}

}  // namespace rg
