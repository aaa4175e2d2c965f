// Standalone timing harness for the CholQR2 panel passes (development tool, not product).
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include tools/cq_bench.cu \
//   paper_conf_hpdc_zhangbw20_b200/csrc/panel_cholqr.cu -o tools/cq_bench
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <algorithm>
#include <vector>
#include <cuda_runtime.h>
// #define RG_CHOL_TRACE 1
#define RG_CF_TRACE 1
#include "../paper_conf_hpdc_zhangbw20_b200/csrc/kernels.h"
namespace rg { thread_local long long g_launches = 0; bool pdl_enabled() { return getenv("RGSQR_NO_PDL") == nullptr; } }
#include "../paper_conf_hpdc_zhangbw20_b200/csrc/panel_cholqr.cu"
template <int NT>
__global__ void chol_nt_kernel(const double* G, double* Rg, float* Rinvg, int reps, long long* cyc) {
    __shared__ __align__(16) double Rs[32 * 34], Ys[32 * 34], Gs[1024];
    for (int e = threadIdx.x; e < 1024; e += NT) Gs[e] = G[e];
    __syncthreads();
    long long t0 = clock64();
    bool ok = true;
    for (int r = 0; r < reps; ++r) ok &= rg::chol_inv_cta<NT, true>(Gs, 32, Rs, Ys, Rg, Rinvg, false);
    long long t1 = clock64();
    if (threadIdx.x == 0) { cyc[0] = (t1 - t0) / reps; cyc[1] = ok; }
}
__global__ void chol_loop_kernel(const double* G, double* Rg, float* Rinvg, int reps, long long* cyc) {
    __shared__ __align__(16) double Rs[32 * 34], Ys[32 * 34];
    long long t0 = clock64();
    bool ok = true;
    for (int r = 0; r < reps; ++r) ok &= rg::chol_inv_cta<256, false>(G, 32, Rs, Ys, Rg, Rinvg, false);
    long long t1 = clock64();
    if (threadIdx.x == 0) { cyc[0] = (t1 - t0) / reps; cyc[1] = ok; }
}
__global__ void dfma_latency_kernel(double* out, int n, long long* cyc) {
    double x = out[threadIdx.x], y = 1.0000001;
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) x = fma(x, y, 1e-9);
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) cyc[2] = (t1 - t0) / n;
    double z = out[threadIdx.x];
    t0 = clock64();
    for (int i = 0; i < n; ++i) z = rsqrt(z + 1.0);
    t1 = clock64();
    out[threadIdx.x + 32] = z;
    if (threadIdx.x == 0) cyc[3] = (t1 - t0) / n;
    t0 = clock64();
    for (int i = 0; i < n; ++i) z = __shfl_sync(0xffffffffu, z, (threadIdx.x + 1) & 31) + 1.0;
    t1 = clock64();
    out[threadIdx.x + 64] = z;
    if (threadIdx.x == 0) cyc[4] = (t1 - t0) / n;
}
int main(int argc, char** argv) {
    const int64_t m = argc > 1 ? atoll(argv[1]) : 65536;
    const int nc = 32;
    std::vector<float> h(m * nc);
    srand(1);
    for (auto& x : h) x = (rand() / (float)RAND_MAX) - 0.5f;
    float *P, *Q, *R; uint16_t* Qh; double* ws; int* flags;
    cudaMalloc(&P, m * nc * 4); cudaMalloc(&Q, m * nc * 4); cudaMalloc(&R, 32 * 32 * 4);
    cudaMalloc(&Qh, m * nc * 2);
    cudaMalloc(&ws, rg::cholqr_ws_doubles(m) * 8); cudaMalloc(&flags, 16384);
    cudaMemset(flags, 0, 16384);
    cudaMemcpy(P, h.data(), m * nc * 4, cudaMemcpyHostToDevice);
    rg::CholqrLaunch L{};
    L.P = P; L.ldp = m; L.Q = Q; L.ldq = m; L.Qh = Qh; L.ldh = m; L.m = m; L.nc = nc; L.ws = ws;
    L.fail = flags; L.counter = flags + 4; L.R = R; L.ldr = 32;
    cudaStream_t st; cudaStreamCreate(&st);
    for (int i = 0; i < 5; ++i) rg::launch_panel_cholqr(L, nullptr, st);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const int iters = 50;
    cudaEventRecord(a, st);
    for (int i = 0; i < iters; ++i) rg::launch_panel_cholqr(L, nullptr, st);
    cudaEventRecord(b, st);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    printf("m=%lld cholqr2 panel: %.2f us per panel (eager launches)\n", (long long)m, ms * 1000 / iters);
    // graph-captured
    cudaGraph_t g; cudaGraphExec_t ge;
    cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
    for (int i = 0; i < iters; ++i) rg::launch_panel_cholqr(L, nullptr, st);
    cudaStreamEndCapture(st, &g);
    cudaGraphInstantiate(&ge, g, 0);
    cudaGraphLaunch(ge, st);
    cudaStreamSynchronize(st);
    cudaEventRecord(a, st);
    cudaGraphLaunch(ge, st);
    cudaEventRecord(b, st);
    cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    printf("m=%lld cholqr2 panel: %.2f us per panel (graph)\n", (long long)m, ms * 1000 / iters);
    // per-pass timing (eager, 50 launches each)
    {
        rg::CqArgs A{};
        A.P = P; A.ldp = m; A.Q = Q; A.ldq = m; A.Qh = Qh; A.ldh = m; A.m = m; A.nc = nc;
        const int grid = rg::cq_grid(m);
        const int ngroups = (grid + rg::CQ_FAN - 1) / rg::CQ_FAN;
        A.ws.part = ws; A.ws.gpart = ws + (size_t)grid * 1024; A.ws.G = A.ws.gpart + (size_t)ngroups * 1024;
        A.ws.R = A.ws.G + 2048; A.ws.Rinv = reinterpret_cast<float*>(A.ws.R + 2048);
        A.ws.counters = flags + 4; A.ws.fail = flags; A.Rout = R; A.ldr = 32;
        for (int pass = 0; pass < 3; ++pass) {
            cudaEventRecord(a, st);
            for (int i = 0; i < iters; ++i) {
                if (pass == 0) rg::cq_pass_kernel<0><<<grid, rg::CQ_THREADS, 0, st>>>(A);
                if (pass == 1) rg::cq_pass_kernel<1><<<grid, rg::CQ_THREADS, 0, st>>>(A);
                if (pass == 2) rg::cq_pass_kernel<2><<<grid, rg::CQ_THREADS, 0, st>>>(A);
            }
            cudaEventRecord(b, st);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            printf("  pass %d: %.2f us\n", pass, ms * 1000 / iters);
        }
        // chol-only kernel timing
        cudaEventRecord(a, st);
        for (int i = 0; i < iters; ++i) rg::cq_factor_kernel<<<1, 256, 0, st>>>(A, 0);
        cudaEventRecord(b, st);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("  chol_inv (1 CTA): %.2f us\n", ms * 1000 / iters);
        A.distributed = 1;
        cudaEventRecord(a, st);
        for (int i = 0; i < iters; ++i) rg::cq_pass_kernel<0><<<grid, rg::CQ_THREADS, 0, st>>>(A);
        cudaEventRecord(b, st);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("  pass 0 without chol (distributed flag): %.2f us\n", ms * 1000 / iters);
    }
    {
        // Cholesky of an SPD 32x32 (identity + small) in a loop: cycles per call
        std::vector<double> G(1024, 0.0);
        for (int i = 0; i < 32; ++i) for (int j = 0; j < 32; ++j) G[i + 32 * j] = (i == j ? 40.0 : 1.0 / (1 + i + j));
        double *dG, *dR, *dout; float* dRi; long long* cyc;
        cudaMalloc(&dG, 8192); cudaMalloc(&dR, 8192); cudaMalloc(&dRi, 4096); cudaMalloc(&cyc, 64); cudaMalloc(&dout, 8192);
        cudaMemcpy(dG, G.data(), 8192, cudaMemcpyHostToDevice);
        cudaMemset(dout, 0, 8192);
        chol_loop_kernel<<<1, 256>>>(dG, dR, dRi, 20, cyc);
        dfma_latency_kernel<<<1, 32>>>(dout, 1000, cyc);
        long long hc[5]; cudaMemcpy(hc, cyc, 40, cudaMemcpyDeviceToHost);
        {   // check R^T R = G and R Rinv = I
            std::vector<double> R(1024); std::vector<float> Ri(1024);
            cudaMemcpy(R.data(), dR, 8192, cudaMemcpyDeviceToHost); cudaMemcpy(Ri.data(), dRi, 4096, cudaMemcpyDeviceToHost);
            double e1 = 0, e2 = 0;
            for (int i = 0; i < 32; ++i) for (int j = 0; j < 32; ++j) {
                double s = 0, t = 0;
                for (int k = 0; k < 32; ++k) { s += R[k + 32 * i] * R[k + 32 * j]; t += R[i + 32 * k] * Ri[k + 32 * j]; }
                e1 = fmax(e1, fabs(s - G[std::min(i, j) + 32 * std::max(i, j)]));
                e2 = fmax(e2, fabs(t - (i == j)));
            }
            printf("  chol check: |R^T R - G| %.2e  |R Rinv - I| %.2e\n", e1, e2);
        }
#ifdef RG_CHOL_TRACE
        {
            long long tr[40]; cudaMemcpyFromSymbol(tr, rg::chol_trace, sizeof(tr));
            printf("  chol step cycles:");
            for (int k = 0; k < 8; ++k) printf(" [p1 %lld bar %lld p2 %lld bar %lld]", tr[10 + k] - tr[k], tr[20 + k] - tr[10 + k], tr[30 + k] - tr[20 + k], tr[k + 1] - tr[30 + k]);
            printf("\n");
        }
#endif
        {
            long long h2[2];
            chol_nt_kernel<32><<<1, 32>>>(dG, dR, dRi, 20, cyc); cudaMemcpy(h2, cyc, 16, cudaMemcpyDeviceToHost);
            printf("  NT=32: %lld cyc;", h2[0]);
            chol_nt_kernel<64><<<1, 64>>>(dG, dR, dRi, 20, cyc); cudaMemcpy(h2, cyc, 16, cudaMemcpyDeviceToHost);
            printf(" NT=64: %lld cyc;", h2[0]);
            chol_nt_kernel<128><<<1, 128>>>(dG, dR, dRi, 20, cyc); cudaMemcpy(h2, cyc, 16, cudaMemcpyDeviceToHost);
            printf(" NT=128: %lld cyc;", h2[0]);
            chol_nt_kernel<256><<<1, 256>>>(dG, dR, dRi, getenv("CHOL_REPS") ? atoi(getenv("CHOL_REPS")) : 20, cyc); cudaMemcpy(h2, cyc, 16, cudaMemcpyDeviceToHost);
            printf(" NT=256: %lld cyc;", h2[0]);
            chol_nt_kernel<512><<<1, 512>>>(dG, dR, dRi, 20, cyc); cudaMemcpy(h2, cyc, 16, cudaMemcpyDeviceToHost);
            printf(" NT=512: %lld cyc;", h2[0]);
            chol_nt_kernel<1024><<<1, 1024>>>(dG, dR, dRi, 20, cyc); cudaMemcpy(h2, cyc, 16, cudaMemcpyDeviceToHost);
            printf(" NT=1024: %lld cyc\n", h2[0]);
        }
        printf("  chol_inv_cta: %lld cycles/call (ok=%lld); DFMA latency %lld cyc; rsqrt(f64) %lld cyc; shfl+DADD %lld cyc\n",
               hc[0], hc[1], hc[2], hc[3], hc[4]);
    }
    {
        unsigned long long tr[16];
        rg::launch_panel_cholqr(L, nullptr, st);
        cudaStreamSynchronize(st);
        cudaMemcpyFromSymbol(tr, rg::cf_trace, sizeof(tr));
        printf("  32-col trace (us): load %.2f gram %.2f allreduce %.2f chol %.2f apply %.2f panel %.2f store %.2f\n",
               (tr[1] - tr[0]) / 1e3, (tr[4] - tr[0]) / 1e3, (tr[5] - tr[0]) / 1e3, (tr[6] - tr[0]) / 1e3,
               (tr[7] - tr[0]) / 1e3, (tr[2] - tr[0]) / 1e3, (tr[3] - tr[0]) / 1e3);
    }
    {
        // two-panel kernel (64 columns), eager back-to-back launches
        float *P2, *Q2, *R2; uint16_t* Qh2;
        cudaMalloc(&P2, (size_t)m * 64 * 4); cudaMalloc(&Q2, (size_t)m * 64 * 4); cudaMalloc(&R2, 64 * 64 * 4);
        cudaMalloc(&Qh2, (size_t)m * 64 * 2);
        std::vector<float> h2((size_t)m * 64);
        for (size_t i = 0; i < h2.size(); ++i) {   // N(0,1) via Box-Muller on a 64-bit hash
            uint64_t z = i * 0x9E3779B97F4A7C15ull + 12345;
            z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
            const double u1 = ((z >> 11) + 1.0) / 9007199254740993.0, u2 = (double)(z & 0x7FF) / 2048.0;
            h2[i] = (float)(sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2));
        }
        cudaMemcpy(P2, h2.data(), h2.size() * 4, cudaMemcpyHostToDevice);
        rg::CholqrLaunch L2 = L;
        L2.P = P2; L2.ldp = m; L2.Q = Q2; L2.ldq = m; L2.Qh = Qh2; L2.ldh = m; L2.nc = 64; L2.R = R2; L2.ldr = 64;
        for (int i = 0; i < 3; ++i) rg::launch_panel_pair(L2, st);
        cudaEventRecord(a, st);
        for (int i = 0; i < iters; ++i) rg::launch_panel_pair(L2, st);
        cudaEventRecord(b, st);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("  64-column kernel: %.2f us, err %s\n", ms * 1000 / iters, cudaGetErrorString(cudaGetLastError()));
        unsigned long long tr[16];
        cudaMemcpyFromSymbol(tr, rg::cf_trace, sizeof(tr));
        printf("  64-col trace (us): load %.2f panel %.2f store %.2f\n",
               (tr[1] - tr[0]) / 1e3, (tr[2] - tr[0]) / 1e3, (tr[3] - tr[0]) / 1e3);
        printf("  pass 0: gram %.2f allreduce %.2f chol %.2f apply %.2f | pass 1 apply %.2f\n", (tr[4] - tr[0]) / 1e3,
               (tr[5] - tr[0]) / 1e3, (tr[6] - tr[0]) / 1e3, (tr[7] - tr[0]) / 1e3, (tr[11] - tr[0]) / 1e3);
    }
    int fl; cudaMemcpy(&fl, flags, 4, cudaMemcpyDeviceToHost);
    printf("fail flag %d, err %s\n", fl, cudaGetErrorString(cudaGetLastError()));
    return 0;
}
