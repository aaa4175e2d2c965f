// Warp-register 32 x 32 Cholesky: cost inside a divergent `if (warp == 0)` region vs a 32-thread
// block vs all warps running it redundantly (development probe).
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/wchol_probe.cu -o tools/wchol_probe
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void wchol32(float* W, int lane, bool write) {
    float c[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) c[i] = W[i * 33 + lane];
#pragma unroll
    for (int k = 0; k < 32; ++k) {
        const float p = __shfl_sync(0xffffffffu, c[k], k);
        float rs = rsqrtf(fmaxf(p, 1e-30f));
        rs = rs * fmaf(-0.5f * p * rs, rs, 1.5f);
        const float r = c[k] * rs;
        c[k] = r;
#pragma unroll
        for (int i = k + 1; i < 32; ++i) c[i] = fmaf(-__shfl_sync(0xffffffffu, r, i), r, c[i]);
    }
    if (write) {
#pragma unroll
        for (int i = 0; i < 32; ++i) W[i * 33 + lane] = c[i];
    }
}

template <int MODE>
__global__ void k(float* g, long long* out) {
    __shared__ float W[32 * 33];
    for (int e = threadIdx.x; e < 32 * 32; e += blockDim.x) {
        const int i = e >> 5, j = e & 31;
        W[i * 33 + j] = (i == j ? 40.f : 0.f) + g[e];
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    long long t0 = clock64();
    if (MODE == 0) wchol32(W, lane, true);                       // 32-thread block
    if (MODE == 1) { if (warp == 0) wchol32(W, lane, true); }    // divergent region
    if (MODE == 2) wchol32(W, lane, warp == 0);                   // every warp, warp 0 writes
    if (MODE == 3) { if (warp < 4) wchol32(W, lane, warp == 0); } // 4 warps
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0) out[MODE] = t1 - t0;
    if (threadIdx.x == 0) g[2048 + MODE] = W[31 * 33 + 31];
}

int main() {
    float* g; long long* o;
    cudaMalloc(&g, 8192 * 4); cudaMalloc(&o, 64);
    float h[1024];
    for (int i = 0; i < 1024; ++i) h[i] = ((i * 37) % 17) * 0.01f;
    for (int i = 0; i < 32; ++i) for (int j = 0; j < 32; ++j) h[i * 32 + j] = h[j * 32 + i] = ((i + j) % 7) * 0.01f;
    cudaMemcpy(g, h, 4096, cudaMemcpyHostToDevice);
    for (int rep = 0; rep < 2; ++rep) {
        k<0><<<1, 32>>>(g, o); k<1><<<1, 512>>>(g, o); k<2><<<1, 512>>>(g, o); k<3><<<1, 512>>>(g, o);
        cudaDeviceSynchronize();
    }
    long long ho[4]; cudaMemcpy(ho, o, 32, cudaMemcpyDeviceToHost);
    printf("wchol32 cycles: 32-thread block %lld, if(warp==0) of 512 %lld, all 16 warps %lld, warps<4 %lld (%s)\n",
           ho[0], ho[1], ho[2], ho[3], cudaGetErrorString(cudaGetLastError()));
    return 0;
}
