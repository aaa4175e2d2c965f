// HBM read bandwidth of a column-major m x 256 fp32 matrix read in row blocks (R rows x 256
// columns per request wave, the tall Gram / apply pattern) vs a contiguous stream (development probe).
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/colread_probe.cu -o tools/colread_probe
#include <cstdio>
#include <cuda_runtime.h>

// each CTA takes row blocks of R rows (grid-strided); within a block, warp w / lane read float4s
template <int R>
__global__ void rowblock(const float* __restrict__ X, long m, int n, float* out, int contiguous_cta) {
    float acc = 0.f;
    const long nblk = m / R;
    if (contiguous_cta) {
        // CTA b owns rows [b m / G, (b + 1) m / G), walks them in blocks of R rows
        const long per = nblk / gridDim.x;
        for (long bi = blockIdx.x * per; bi < (blockIdx.x + 1) * per; ++bi)
            for (int e = threadIdx.x; e < R / 4 * n; e += blockDim.x) {
                const int c = e / (R / 4), q = e % (R / 4);
                const float4 v = __ldcs(reinterpret_cast<const float4*>(X + bi * R + 4 * q + (long)c * m));
                acc += v.x + v.y + v.z + v.w;
            }
    } else {
        for (long bi = blockIdx.x; bi < nblk; bi += gridDim.x)
            for (int e = threadIdx.x; e < R / 4 * n; e += blockDim.x) {
                const int c = e / (R / 4), q = e % (R / 4);
                const float4 v = __ldcs(reinterpret_cast<const float4*>(X + bi * R + 4 * q + (long)c * m));
                acc += v.x + v.y + v.z + v.w;
            }
    }
    if (acc == 12345.f) out[0] = acc;
}
__global__ void stream(const float4* __restrict__ X, long n4, float* out) {
    float acc = 0.f;
    for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n4; i += (long)gridDim.x * blockDim.x) {
        const float4 v = __ldcs(X + i);
        acc += v.x + v.y + v.z + v.w;
    }
    if (acc == 12345.f) out[0] = acc;
}
int main() {
    const long m = 2097152; const int n = 256;
    float* X; float* o;
    cudaMalloc(&X, m * n * 4); cudaMalloc(&o, 64);
    cudaMemset(X, 0, m * n * 4);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto run = [&](const char* name, auto f) {
        float best = 1e9;
        for (int i = 0; i < 5; ++i) {
            cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
        }
        printf("%-44s %.3f ms  %.2f TB/s (%s)\n", name, best, m * n * 4.0 / (best * 1e-3) / 1e12, cudaGetErrorString(cudaGetLastError()));
    };
    run("contiguous stream (148 x 8 CTAs)", [&] { stream<<<148 * 8, 512>>>((const float4*)X, m * n / 4, o); });
    run("row blocks of 32 (strided over CTAs)", [&] { rowblock<32><<<148 * 4, 512>>>(X, m, n, o, 0); });
    run("row blocks of 64 (strided)", [&] { rowblock<64><<<148 * 4, 512>>>(X, m, n, o, 0); });
    run("row blocks of 128 (strided)", [&] { rowblock<128><<<148 * 4, 512>>>(X, m, n, o, 0); });
    run("row blocks of 512 (strided)", [&] { rowblock<512><<<148 * 4, 512>>>(X, m, n, o, 0); });
    run("row blocks of 64 (contiguous per CTA)", [&] { rowblock<64><<<148 * 4, 512>>>(X, m, n, o, 1); });
    run("row blocks of 512 (contiguous per CTA)", [&] { rowblock<512><<<148 * 4, 512>>>(X, m, n, o, 1); });
    return 0;
}
