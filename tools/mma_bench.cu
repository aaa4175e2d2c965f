// Microbenchmark (development tool): legacy mma.sync throughput per SM on sm_100a.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/mma_bench.cu -o tools/mma_bench
#include <cstdio>
#include <cuda_runtime.h>
template <int KIND>
__global__ void k(float* out, long long* cyc, int iters) {
    float d[8][4] = {};
    double dd[8][2] = {};
    unsigned a0 = threadIdx.x, a1 = a0 * 3, a2 = a0 * 5, a3 = a0 * 7, b0 = a0 * 11, b1 = a0 * 13;
    double fa = threadIdx.x * 1e-3, fb = fa + 1;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            if (KIND == 0)
                asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                             : "+f"(d[u][0]), "+f"(d[u][1]), "+f"(d[u][2]), "+f"(d[u][3])
                             : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
            else if (KIND == 1)
                asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                             : "+f"(d[u][0]), "+f"(d[u][1]), "+f"(d[u][2]), "+f"(d[u][3])
                             : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
            else
                asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                             : "+d"(dd[u][0]), "+d"(dd[u][1]) : "d"(fa), "d"(fb));
        }
    }
    long long t1 = clock64();
    float s = 0;
    for (int u = 0; u < 8; ++u) s += d[u][0] + d[u][1] + d[u][2] + d[u][3] + (float)dd[u][0] + (float)dd[u][1];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
int main() {
    float* out; long long* cyc;
    cudaMalloc(&out, 148 * 1024 * 4); cudaMalloc(&cyc, 148 * 8);
    const int iters = 2000;
    const char* names[3] = {"f16 m16n8k16", "tf32 m16n8k8", "f64 m8n8k4"};
    const double fma_per[3] = {16 * 8 * 16, 16 * 8 * 8, 8 * 8 * 4};
    for (int kind = 0; kind < 3; ++kind)
        for (int warps : {4, 8, 16, 32}) {
            auto kern = kind == 0 ? k<0> : kind == 1 ? k<1> : k<2>;
            kern<<<148, warps * 32>>>(out, cyc, 10);
            kern<<<148, warps * 32>>>(out, cyc, iters);
            cudaDeviceSynchronize();
            long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
            double per_clk = (double)warps * iters * 8 * fma_per[kind] / c;
            printf("%-14s warps %2d: %.1f FMA/clk/SM (%.0f cycles)\n", names[kind], warps, per_clk, (double)c);
        }
    return 0;
}
