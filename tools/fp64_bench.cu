// microbenchmark: fp64 DFMA / F2F / DMMA throughput per SM on this GPU (development tool)
#include <cstdio>
#include <cuda_runtime.h>
__global__ void dfma_tp(double* out, int n) {
    double a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
    const double b = 1.0000001, c = 1e-9;
    for (int i = 0; i < n; ++i) {
        a0 = fma(a0, b, c); a1 = fma(a1, b, c); a2 = fma(a2, b, c); a3 = fma(a3, b, c);
        a4 = fma(a4, b, c); a5 = fma(a5, b, c); a6 = fma(a6, b, c); a7 = fma(a7, b, c);
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7;
}
__global__ void f2f_tp(double* out, const float* in, int n) {
    float x0 = in[threadIdx.x], x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3;
    double s0 = 0, s1 = 0, s2 = 0, s3 = 0;
    for (int i = 0; i < n; ++i) {
        s0 += (double)x0; s1 += (double)x1; s2 += (double)x2; s3 += (double)x3;
        x0 += 1.f; x1 += 1.f; x2 += 1.f; x3 += 1.f;
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = s0 + s1 + s2 + s3;
}
__global__ void dmma_tp(double* out, int n) {
    double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
    double c0 = 0, c1 = 0, d0 = 0, d1 = 0, e0 = 0, e1 = 0, f0 = 0, f1 = 0;
    for (int i = 0; i < n; ++i) {
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};" : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};" : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};" : "+d"(e0), "+d"(e1) : "d"(a), "d"(b));
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};" : "+d"(f0), "+d"(f1) : "d"(a), "d"(b));
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = c0 + c1 + d0 + d1 + e0 + e1 + f0 + f1;
}
// larger fp64 shapes (sm_90+): m16n8k4 (A 2 regs, B 1, C 4), m16n8k8 (A 4, B 2), m16n8k16 (A 8, B 4)
__global__ void dmma16_tp(double* out, int n) {
    double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
    double c[4][4] = {};
    for (int i = 0; i < n; ++i) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
            asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                         : "+d"(c[u][0]), "+d"(c[u][1]), "+d"(c[u][2]), "+d"(c[u][3]) : "d"(a), "d"(a), "d"(b));
    }
    double s = 0; for (int u = 0; u < 4; ++u) for (int v = 0; v < 4; ++v) s += c[u][v];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void dmma16k16_tp(double* out, int n) {
    double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
    double c[4][4] = {};
    for (int i = 0; i < n; ++i) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
            asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};"
                         : "+d"(c[u][0]), "+d"(c[u][1]), "+d"(c[u][2]), "+d"(c[u][3])
                         : "d"(a), "d"(a), "d"(a), "d"(a), "d"(a), "d"(a), "d"(a), "d"(a), "d"(b), "d"(b), "d"(b), "d"(b));
    }
    double s = 0; for (int u = 0; u < 4; ++u) for (int v = 0; v < 4; ++v) s += c[u][v];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// mma.sync m16n8k16 f16 -> f32: throughput (4 independent accumulators) and latency (1 chain)
__global__ void hmma_tp(float* out, int n, int chains) {
    unsigned a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, b0 = a0 ^ 5, b1 = a0 ^ 7;
    float c[4][4] = {};
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) {
        if (chains == 4) {
#pragma unroll
            for (int u = 0; u < 4; ++u)
                asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                             : "+f"(c[u][0]), "+f"(c[u][1]), "+f"(c[u][2]), "+f"(c[u][3]) : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
        } else {
            asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                         : "+f"(c[0][0]), "+f"(c[0][1]), "+f"(c[0][2]), "+f"(c[0][3]) : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
        }
    }
    long long t1 = clock64();
    float s = 0; for (int u = 0; u < 4; ++u) for (int v = 0; v < 4; ++v) s += c[u][v];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s + (threadIdx.x == 0 && blockIdx.x == 0 ? (float)(t1 - t0) : 0.f);
}
int main() {
    double* out; float* in;
    cudaMalloc(&out, 148 * 1024 * 8 * 4); cudaMalloc(&in, 4096);
    cudaMemset(in, 0, 4096);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float ms;
    const int n = 4096;
    dfma_tp<<<148 * 4, 256>>>(out, 16);
    cudaEventRecord(a); dfma_tp<<<148 * 4, 256>>>(out, n); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    double fl = 148.0 * 4 * 256 * n * 8;
    printf("DFMA: %.2f TFMA/s -> %.1f DFMA/clk/SM @1.9GHz\n", fl / ms / 1e9, fl / ms / 1e-3 / 148 / 1.9e9);
    cudaEventRecord(a); f2f_tp<<<148 * 4, 256>>>(out, in, n); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    fl = 148.0 * 4 * 256 * n * 4;
    printf("F2F.F64.F32 (+DADD): %.2f T/s -> %.1f /clk/SM\n", fl / ms / 1e9, fl / ms / 1e-3 / 148 / 1.9e9);
    cudaEventRecord(a); dmma_tp<<<148 * 4, 256>>>(out, n); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    fl = 148.0 * 4 * 8 * n * 4 * 256;   // warps * mma * 256 FMA
    printf("DMMA m8n8k4: %.2f TFMA/s -> %.1f FMA/clk/SM (%s)\n", fl / ms / 1e9, fl / ms / 1e-3 / 148 / 1.9e9,
           cudaGetErrorString(cudaGetLastError()));
    cudaEventRecord(a); dmma16_tp<<<148 * 4, 256>>>(out, n); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    fl = 148.0 * 4 * 8 * n * 4 * 512;
    printf("DMMA m16n8k4: %.2f TFMA/s -> %.1f FMA/clk/SM (%s)\n", fl / ms / 1e9, fl / ms / 1e-3 / 148 / 1.9e9,
           cudaGetErrorString(cudaGetLastError()));
    cudaEventRecord(a); dmma16k16_tp<<<148 * 4, 256>>>(out, n / 4); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    fl = 148.0 * 4 * 8 * (n / 4) * 4 * 2048;
    printf("DMMA m16n8k16: %.2f TFMA/s -> %.1f FMA/clk/SM (%s)\n", fl / ms / 1e9, fl / ms / 1e-3 / 148 / 1.9e9,
           cudaGetErrorString(cudaGetLastError()));
    {
        float* fo; cudaMalloc(&fo, 148 * 1024 * 4 * 4);
        hmma_tp<<<148 * 4, 256>>>(fo, 64, 4);
        cudaEventRecord(a); hmma_tp<<<148 * 4, 256>>>(fo, n, 4); cudaEventRecord(b); cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        fl = 148.0 * 4 * 8 * n * 4 * 4096.0;   // warps * mma * (16*8*16*2 flops)
        printf("HMMA m16n8k16 (mma.sync): %.1f TFLOP/s -> %.0f flop/clk/SM\n", fl / ms / 1e9, fl / ms / 1e-3 / 148 / 1.9e9);
        hmma_tp<<<1, 32>>>(fo, 4096, 1);
        float h0; cudaMemcpy(&h0, fo, 4, cudaMemcpyDeviceToHost);
        printf("HMMA dependent-chain latency: %.1f cycles per mma\n", h0 / 4096.0);
    }
    return 0;
}
