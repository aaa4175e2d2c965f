// Standalone timing of the small Jacobi SVD (development tool, not product).
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/jacobi_bench.cu -o tools/jacobi_bench
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <vector>
#include <cuda_runtime.h>
#include "../paper_conf_hpdc_zhangbw20_b200/csrc/kernels.h"
namespace rg { thread_local long long g_launches = 0; bool pdl_enabled() { return false; } }
#include "../paper_conf_hpdc_zhangbw20_b200/csrc/lowrank.cu"
int main(int argc, char** argv) {
    const int l = argc > 1 ? atoi(argv[1]) : 528;
    const int r = l - 16;
    // upper-triangular R with a geometric-ish spectrum: R = triu(random) * diag decay
    std::vector<float> R((size_t)l * l, 0.f);
    srand(3);
    for (int j = 0; j < l; ++j)
        for (int i = 0; i <= j; ++i)
            R[i + (size_t)j * l] = ((rand() / (float)RAND_MAX) - 0.5f) * powf(10.f, -3.f * j / l) + (i == j ? 2.f * powf(10.f, -3.f * j / l) : 0.f);
    float *dR, *S, *Ub, *Vb; double *W, *V, *sig; int* flags;
    cudaMalloc(&dR, R.size() * 4); cudaMalloc(&S, l * 4); cudaMalloc(&Ub, (size_t)l * l * 4); cudaMalloc(&Vb, (size_t)l * l * 4);
    cudaMalloc(&W, (size_t)l * l * 8); cudaMalloc(&V, (size_t)l * l * 8); cudaMalloc(&sig, l * 8); cudaMalloc(&flags, 64);
    cudaMemcpy(dR, R.data(), R.size() * 4, cudaMemcpyHostToDevice);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int it = 0; it < 3; ++it) {
        cudaEventRecord(a);
        cudaError_t e = rg::launch_jacobi_svd(dR, l, l, r, W, V, sig, flags, S, Ub, Vb, 0);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        int hf[2]; cudaMemcpy(hf, flags, 8, cudaMemcpyDeviceToHost);
        printf("l=%d: %.3f ms, sweeps %d (%s / %s)\n", l, ms, hf[1], cudaGetErrorString(e), cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
