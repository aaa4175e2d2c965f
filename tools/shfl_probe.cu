// Latency / throughput probe for the warp-register Cholesky of the leaf (development tool).
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/shfl_probe.cu -o tools/shfl_probe
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ float rcp32(float x) {
    float y;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

__global__ void probe(long long* out, float* sink, float seed) {
    const int lane = threadIdx.x & 31;
    float v = seed + lane;
    long long t0, t1;
    // (1) dependent SHFL.IDX chain
    __syncwarp();
    t0 = clock64();
#pragma unroll
    for (int i = 0; i < 64; ++i) v = __shfl_sync(0xffffffffu, v, (i * 7) & 31);
    t1 = clock64();
    if (lane == 0 && threadIdx.x == 0) out[0] = (t1 - t0);
    // (2) independent SHFL.IDX (throughput, one warp)
    float a[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) a[i] = v + i;
    __syncwarp();
    t0 = clock64();
#pragma unroll
    for (int r = 0; r < 8; ++r)
#pragma unroll
        for (int i = 0; i < 16; ++i) a[i] = __shfl_sync(0xffffffffu, a[i], (i + r) & 31);
    t1 = clock64();
    if (threadIdx.x == 0) out[1] = (t1 - t0);
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += a[i];
    // (3) dependent MUFU.RCP chain
    __syncwarp();
    t0 = clock64();
#pragma unroll
    for (int i = 0; i < 64; ++i) s = rcp32(s + 1.f);
    t1 = clock64();
    if (threadIdx.x == 0) out[2] = (t1 - t0);
    // (4) 32 x 32 LDL in registers (the leaf's lf_wldl32)
    float c[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) c[i] = (i == lane) ? 40.f : 1.f / (1 + i + lane);
    __syncwarp();
    t0 = clock64();
#pragma unroll
    for (int k = 0; k < 32; ++k) {
        const float d = __shfl_sync(0xffffffffu, c[k], k);
        const float t = c[k] * rcp32(d);
#pragma unroll
        for (int i = k + 1; i < 32; ++i) c[i] = fmaf(-__shfl_sync(0xffffffffu, c[k], i), t, c[i]);
    }
    t1 = clock64();
    if (threadIdx.x == 0) out[3] = (t1 - t0);
#pragma unroll
    for (int i = 0; i < 32; ++i) s += c[i];
    sink[threadIdx.x + blockIdx.x * blockDim.x] = s + v;
}


constexpr int BR = 36;
__device__ __forceinline__ void rot_step(float (&x)[32], const float (&rv)[32], float ri) {
    const float tx = x[0] * ri;
#pragma unroll
    for (int i = 1; i < 32; ++i) x[i - 1] = fmaf(-rv[i], tx, x[i]);
    x[31] = 0.f;
}
__global__ void lead_probe(long long* out, float* sink) {
    __shared__ __align__(16) float Urot[32 * BR];
    __shared__ __align__(16) float Xo[32 * BR];
    const int lane = threadIdx.x & 31;
    float c[32], x[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) {
        c[i] = (i == lane) ? 40.f : 1.f / (1 + i + lane);
        x[i] = 1.f / (2 + i + lane);
    }
    float dk = 0.f;
    __syncthreads();
    long long t0 = clock64();
    if (threadIdx.x < 32) {
#pragma unroll 1
        for (int k = 0; k < 32; ++k) {
            float* row = Urot + k * BR;
            row[(lane - k) & 31] = c[0];
            Xo[k * BR + lane] = x[0];
            __syncwarp();
            float rv[32];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const float4 v = *reinterpret_cast<const float4*>(row + 4 * q);
                rv[4 * q] = v.x; rv[4 * q + 1] = v.y; rv[4 * q + 2] = v.z; rv[4 * q + 3] = v.w;
            }
            if (lane == k) dk = rv[0];
            const float ri = rcp32(rv[0]);
            rot_step(c, rv, ri);
            rot_step(x, rv, ri);
        }
    }
    long long t1 = clock64();
    __syncthreads();
    if (threadIdx.x == 0) out[4] = t1 - t0;
    float s = dk;
#pragma unroll
    for (int i = 0; i < 32; ++i) s += c[i] + x[i];
    sink[threadIdx.x] = s + Urot[threadIdx.x % (32 * BR)] + Xo[threadIdx.x];
}

int main() {
    long long* d;
    float* sink;
    cudaMalloc(&d, 64);
    cudaMalloc(&sink, 1 << 20);
    for (int threads : {32, 512}) {
        for (int rep = 0; rep < 3; ++rep) probe<<<1, threads>>>(d, sink, 1.f);
        long long h[4];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        printf("threads %d: SHFL dep %.1f cyc, SHFL indep %.2f cyc/instr, RCP dep %.1f cyc, LDL32 %lld cyc (%.0f / pivot)\n",
               threads, h[0] / 64.0, h[1] / 128.0, h[2] / 64.0, h[3], h[3] / 32.0);
    }
    for (int threads : {32, 512}) {
        for (int rep = 0; rep < 3; ++rep) lead_probe<<<1, threads>>>(d, sink);
        long long h[5];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        printf("threads %d: lead32 (smem row broadcast, rotated, rolled loop) %lld cyc (%.0f / step)\n", threads, h[4], h[4] / 32.0);
    }
    return 0;
}
