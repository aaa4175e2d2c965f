// Standalone timing + check of the tall Cholesky / inverse kernel (tall.cu tl_chol_kernel), development tool.
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include tools/tchol_bench.cu -o tools/tchol_bench
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cmath>
#include <cuda_runtime.h>
#include "../paper_conf_hpdc_zhangbw20_b200/csrc/kernels.h"
namespace rg {
thread_local long long g_launches = 0;
bool pdl_enabled() { return false; }
int dev_sms() { int d = 0, v = 0; cudaGetDevice(&d); cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d); return v; }
int dev_smem_optin() { return 232448; }
cudaError_t ensure_smem_attr(const void* k, size_t b) { return cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)b); }
}
#include "../paper_conf_hpdc_zhangbw20_b200/csrc/tall.cu"
int main(int argc, char** argv) {
    const int n = argc > 1 ? atoi(argv[1]) : 256;
    const double off = argc > 2 ? atof(argv[2]) : 1e-3;
    std::vector<double> B((size_t)n * n), G((size_t)n * n, 0.0);
    srand(3);
    for (int i = 0; i < n; ++i)
        for (int j = 0; j < n; ++j) B[i + (size_t)j * n] = (i == j ? 1.0 : 0.0) + off * ((rand() / (double)RAND_MAX) - 0.5);
    for (int i = 0; i < n; ++i)
        for (int j = 0; j < n; ++j) {
            double s = 0;
            for (int k = 0; k < n; ++k) s += B[k + (size_t)i * n] * B[k + (size_t)j * n];
            G[i + (size_t)j * n] = s * (1.0 + 0.5 * ((i * 7) % 5));   // unequal column norms
        }
    for (int i = 0; i < n; ++i)
        for (int j = 0; j < n; ++j) G[i + (size_t)j * n] = G[j + (size_t)i * n] = sqrt(G[i + (size_t)i * n] * 0 + 1) * G[std::min(i, j) + (size_t)std::max(i, j) * n];
    double* dG; float* R; void* ws;
    cudaMalloc(&dG, n * n * 8); cudaMalloc(&R, n * n * 4); cudaMalloc(&ws, rg::tall_ws_bytes()); cudaMemset(ws, 0, rg::tall_ws_bytes());
    cudaMemcpy(dG, G.data(), n * n * 8, cudaMemcpyHostToDevice);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float best = 1e9;
    for (int it = 0; it < 20; ++it) {
        cudaEventRecord(a);
        rg::launch_tall_chol_apply(nullptr, 1, 0, n, dG, 1.0, 1.0f, 1, 1e9, R, n, ws, 0);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    std::vector<float> hR((size_t)n * n), hX((size_t)256 * 256);
    cudaMemcpy(hR.data(), R, n * n * 4, cudaMemcpyDeviceToHost);
    // R^-1 (scaled) from the workspace: rinv is the first TL_N^2 floats of the tail
    double err = 0, nrm = 0;
    for (int i = 0; i < n; ++i)
        for (int j = i; j < n; ++j) {
            double s = 0;
            for (int k = 0; k <= i; ++k) s += (double)hR[k + (size_t)i * n] * hR[k + (size_t)j * n];
            err = fmax(err, fabs(s - G[i + (size_t)j * n]));
            nrm = fmax(nrm, fabs(G[i + (size_t)j * n]));
        }
    int flag; double k[2];
    cudaMemcpy(&flag, rg::tall_flag(ws), 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(k, rg::tall_kout(ws), 16, cudaMemcpyDeviceToHost);
    printf("n=%d off=%g: chol+inverse %.1f us, max|R^T R - G|/max|G| = %.2e, flag %d kappa %.4g (%s)\n", n, off, best * 1e3,
           err / nrm, flag, k[0], cudaGetErrorString(cudaGetLastError()));
    return 0;
}
