// Standalone timing harness for the leaf kernel (development tool, not product).
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include tools/leaf_bench.cu -o tools/leaf_bench
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cmath>
#define LF_TRACE 1
#include "../paper_conf_hpdc_zhangbw20_b200/csrc/kernels.h"
namespace rg {
thread_local long long g_launches = 0;
bool pdl_enabled() { return false; }
int dev_sms() { int d = 0, v = 0; cudaGetDevice(&d); cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d); return v; }
int dev_smem_optin() { int d = 0, v = 0; cudaGetDevice(&d); cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, d); return v; }
cudaError_t ensure_smem_attr(const void* k, size_t b) { return cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)b); }
}
#include "../paper_conf_hpdc_zhangbw20_b200/csrc/leaf.cu"
__global__ void lat_probe(long long* cyc, double* out, int n) {
    __shared__ double sm[1024];
    __shared__ int chase[64];
    const int lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) sm[i] = 1.0 + i * 1e-9;
    for (int i = threadIdx.x; i < 64; i += blockDim.x) chase[i] = (i + 1) & 63;
    __syncthreads();
    if (threadIdx.x >= 32) return;
    double a0 = out[lane], a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
    const double b = 1.0000001, c = 1e-9;
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) {
        a0 = fma(a0, b, c); a1 = fma(a1, b, c); a2 = fma(a2, b, c); a3 = fma(a3, b, c);
        a4 = fma(a4, b, c); a5 = fma(a5, b, c); a6 = fma(a6, b, c); a7 = fma(a7, b, c);
    }
    long long t1 = clock64();
    for (int i = 0; i < n; ++i) a0 = fma(a0, b, c);
    long long t2 = clock64();
    int p = lane & 63;
    for (int i = 0; i < n; ++i) p = chase[p];
    long long t3 = clock64();
    double v = 0;
    for (int i = 0; i < n; ++i) {
        sm[(i & 31) * 32 + lane] = v + lane;
        __syncwarp();
        v = sm[(i & 31) * 32 + ((lane + 1) & 31)];
    }
    long long t4 = clock64();
    float f0 = (float)a1, f1 = f0 + 1, f2 = f0 + 2, f3 = f0 + 3, f4 = f0 + 4, f5 = f0 + 5, f6 = f0 + 6, f7 = f0 + 7;
    for (int i = 0; i < n; ++i) {
        f0 = fmaf(f0, 1.0001f, 1e-7f); f1 = fmaf(f1, 1.0001f, 1e-7f); f2 = fmaf(f2, 1.0001f, 1e-7f); f3 = fmaf(f3, 1.0001f, 1e-7f);
        f4 = fmaf(f4, 1.0001f, 1e-7f); f5 = fmaf(f5, 1.0001f, 1e-7f); f6 = fmaf(f6, 1.0001f, 1e-7f); f7 = fmaf(f7, 1.0001f, 1e-7f);
    }
    long long t5 = clock64();
    double r = a2;
    for (int i = 0; i < n; ++i) r = rg::lf_rsqrt(r + 2.0);
    long long t6 = clock64();
    out[lane] = a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 + p + v + f0 + f1 + f2 + f3 + f4 + f5 + f6 + f7 + r;
    if (lane == 0) {
        cyc[0] = (t1 - t0) * 100 / (8 * n); cyc[1] = (t2 - t1) * 100 / n; cyc[2] = (t3 - t2) * 100 / n;
        cyc[3] = (t4 - t3) * 100 / n; cyc[4] = (t5 - t4) * 100 / (8 * n); cyc[5] = (t6 - t5) * 100 / n;
    }
}
__global__ void __launch_bounds__(512, 1) chol64_probe(long long* cyc, int reps) {
    extern __shared__ __align__(16) uint8_t sm[];
    rg::LfSmem s(sm, 36);
    for (int e = threadIdx.x; e < 4096; e += blockDim.x) {
        const int i = e >> 6, j = e & 63;
        s.G[i * rg::LF_GLD + j] = (i == j ? 80.0 : 1.0 / (1 + i + j));
        if (i == j) s.gdiag[i] = 80.0;
    }
    __syncthreads();
    long long t0 = clock64(), t1 = 0;
    int bad = 0;
    for (int r = 0; r < reps; ++r) {
        if (threadIdx.x < 128) bad += rg::lf_chol(s);
        __syncthreads();
        if (r == 0) {
            t1 = clock64();
            if (threadIdx.x == 0) {   // check R^T R == G
                double err = 0;
                for (int i = 0; i < 64; ++i)
                    for (int j = i; j < 64; ++j) {
                        double acc = 0;
                        for (int k = 0; k <= i; ++k) acc += s.Rs[k * rg::LF_GLD + i] * s.Rs[k * rg::LF_GLD + j];
                        const double g = (i == j ? 80.0 : 1.0 / (1 + i + j));
                        err = fmax(err, fabs(acc - g) / 80.0);
                    }
                cyc[5] = (long long)(err * 1e18);
            }
            __syncthreads();
        }
        for (int e = threadIdx.x; e < 4096; e += blockDim.x) {
            const int i = e >> 6, j = e & 63;
            s.G[i * rg::LF_GLD + j] = (i == j ? 80.0 : 1.0 / (1 + i + j));
        }
        __syncthreads();
    }
    long long t2 = clock64();
    if (threadIdx.x == 0) { cyc[2] = t1 - t0; cyc[3] = (t2 - t1) / (reps - 1); cyc[4] = bad; }
}
__global__ void bar_probe(long long* cyc, int n) {
    __shared__ double sm[2][64];
    const int t = threadIdx.x;
    double v = 1.0 + t;
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) {
        if (t < 64) sm[i & 1][t] = v;
        __syncthreads();
        v = sm[i & 1][(t + 1) & 63] * 1.0000001;
    }
    long long t1 = clock64();
    if (t < 64) sm[0][t] = v;
    if (t == 0) cyc[blockDim.x == 512 ? 0 : 1] = (t1 - t0) * 100 / n;
}
__global__ void stream_ef(float4* p, size_t n) {   // read-modify-write with L2 evict_first
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        float4 v;
        asm volatile("ld.global.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
                     : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p + i), "l"(pol));
        v.x += 1.f;
        asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;"
                     :: "l"(p + i), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "l"(pol) : "memory");
    }
}
__global__ void stream_plain(float4* p, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        float4 v = p[i];
        v.x += 1.f;
        p[i] = v;
    }
}
int main(int argc, char** argv) {
    {
        long long* cyc; cudaMalloc(&cyc, 64); cudaMemset(cyc, 0, 64);
        bar_probe<<<1, 512>>>(cyc, 4096);
        bar_probe<<<1, 128>>>(cyc, 4096);
        long long hc[2]; cudaMemcpy(hc, cyc, 16, cudaMemcpyDeviceToHost);
        printf("STS+syncthreads+LDS+DMUL chain (cycles x100): 512 threads %lld, 128 threads %lld\n", hc[0], hc[1]);
        size_t smb = 64 * 36 * 4 + rg::LfSmem::fixed_bytes();
        cudaFuncSetAttribute(chol64_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smb);
        chol64_probe<<<1, 512, smb>>>(cyc, 10);
        long long hh[6]; cudaMemcpy(hh, cyc, 48, cudaMemcpyDeviceToHost);
        printf("chol64: first %lld cycles, warm %lld cycles (incl. G rebuild), bad-sum %lld, max|R^T R - G|/80 = %.3g (%s)\n", hh[2], hh[3], hh[4], hh[5] * 1e-18, cudaGetErrorString(cudaGetLastError()));
    }
    {
        long long* cyc; double* out; cudaMalloc(&cyc, 64); cudaMalloc(&out, 1024); cudaMemset(out, 0, 1024);
        lat_probe<<<1, 64>>>(cyc, out, 4096);
        long long hc[6]; cudaMemcpy(hc, cyc, 48, cudaMemcpyDeviceToHost);
        printf("lat probe (cycles x100): DFMA issue %lld, DFMA latency %lld, LDS latency %lld, STS+syncwarp+LDS %lld, FFMA issue %lld, rsqrt(approx+newton) %lld\n",
               hc[0], hc[1], hc[2], hc[3], hc[4], hc[5]);
    }
    const int64_t m = argc > 1 ? atoll(argv[1]) : 65536;
    const int nc = argc > 2 ? atoi(argv[2]) : 64;
    std::vector<float> h((size_t)m * nc);
    srand(1);
    // N(0,1) columns (Box-Muller), scaled like the library's column scaling (norm ~300)
    for (size_t i = 0; i < h.size(); ++i) {
        const double u1 = (rand() + 1.0) / ((double)RAND_MAX + 2.0), u2 = rand() / ((double)RAND_MAX + 1.0);
        const double norm = 256.0 + 256.0 * (double)((i / m) * 37 % 64) / 64.0;   // like the column scaling
        h[i] = (float)(sqrt(-2 * log(u1)) * cos(6.283185307179586 * u2) * norm / sqrt((double)m));
    }
    float *P, *Q, *R; uint16_t* Qh; double* ws; unsigned* bar; int* status;
    cudaMalloc(&P, m * nc * 4); cudaMalloc(&Q, m * nc * 4); cudaMalloc(&R, 64 * 64 * 4);
    cudaMalloc(&Qh, m * nc * 2); cudaMalloc(&ws, rg::leaf_ws_doubles() * 8); cudaMemset(ws, 0, rg::leaf_ws_doubles() * 8); cudaMalloc(&bar, 4096);
    cudaMalloc(&status, 64); cudaMemset(bar, 0, 4096); cudaMemset(status, 0x7f, 64);
    cudaMemcpy(P, h.data(), m * nc * 4, cudaMemcpyHostToDevice);
    rg::LeafLaunch L{};
    L.Q = Q; L.ldq = m; L.Qh = Qh; L.ldh = m; L.m = m; L.nc = nc; L.R = R; L.ldr = 64; L.ws = ws; L.bar = bar;
    L.status = status; L.col0 = 0;
    uint16_t* qa16 = nullptr;
    if (argc > 3 && atoi(argv[3])) {   // prologue with a random 64-column 16-bit Q_A
        std::vector<uint16_t> hq((size_t)m * 64);
        // a nearly orthonormal Q_A: N(0, 1/m) entries as fp16
        for (size_t i = 0; i < hq.size(); ++i) {
            const double u1 = (rand() + 1.0) / ((double)RAND_MAX + 2.0), u2 = rand() / ((double)RAND_MAX + 1.0);
            const __half hv = __float2half((float)(sqrt(-2 * log(u1)) * cos(6.283185307179586 * u2) / sqrt((double)m)));
            hq[i] = *reinterpret_cast<const uint16_t*>(&hv);
        }
        cudaMalloc(&qa16, hq.size() * 2);
        cudaMemcpy(qa16, hq.data(), hq.size() * 2, cudaMemcpyHostToDevice);
        L.pq = qa16; L.ph = 64;
        cudaMalloc(&R, 128 * 64 * 4);
        L.R = R + 64; L.ldr = 128;
    }
    cudaStream_t st; cudaStreamCreate(&st);
    const int iters = 50;
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float tot = 0;
    for (int i = 0; i < iters + 3; ++i) {
        cudaMemcpyAsync(Q, P, m * nc * 4, cudaMemcpyDeviceToDevice, st);
        cudaEventRecord(a, st);
        cudaError_t e = rg::launch_leaf(L, st);
        cudaEventRecord(b, st);
        cudaEventSynchronize(b);
        if (e != cudaSuccess) { printf("launch error %s\n", cudaGetErrorString(e)); return 1; }
        float ms; cudaEventElapsedTime(&ms, a, b);
        if (i >= 3) tot += ms;
    }
    {   // back-to-back launches (code and data warm) vs after a 1 GB L2-flushing memset
        void* big; cudaMalloc(&big, 1ull << 30);
        float t2 = 0, t3 = 0;
        for (int i = 0; i < 13; ++i) {
            cudaMemcpyAsync(Q, P, m * nc * 4, cudaMemcpyDeviceToDevice, st);
            rg::launch_leaf(L, st);
            cudaEventRecord(a, st);
            rg::launch_leaf(L, st);
            cudaEventRecord(b, st);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (i >= 3) t2 += ms;
            cudaMemcpyAsync(Q, P, m * nc * 4, cudaMemcpyDeviceToDevice, st);
            cudaMemsetAsync(big, i, 1ull << 30, st);
            cudaEventRecord(a, st);
            rg::launch_leaf(L, st);
            cudaEventRecord(b, st);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            if (i >= 3) t3 += ms;
        }
        printf("  second back-to-back launch %.2f us; after a 1 GB memset %.2f us\n", t2 * 100, t3 * 100);
        for (int mode = 0; mode < 2; ++mode) {
            float tt = 0;
            for (int i = 0; i < 13; ++i) {
                cudaMemcpyAsync(Q, P, m * nc * 4, cudaMemcpyDeviceToDevice, st);
                if (mode) stream_ef<<<148 * 8, 256, 0, st>>>((float4*)big, (1ull << 30) / 16);
                else stream_plain<<<148 * 8, 256, 0, st>>>((float4*)big, (1ull << 30) / 16);
                cudaEventRecord(a, st);
                rg::launch_leaf(L, st);
                cudaEventRecord(b, st);
                cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b);
                if (i >= 3) tt += ms;
            }
            printf("  after a 1 GB %s read-modify-write stream: %.2f us\n", mode ? "L2-evict_first" : "plain", tt * 100);
        }
        cudaFree(big);
    }
    printf("m=%lld nc=%d leaf kernel: %.2f us (err %s)\n", (long long)m, nc, tot * 1000 / iters,
           cudaGetErrorString(cudaGetLastError()));
    unsigned long long tr[48];
    cudaMemcpyFromSymbol(tr, rg::lf_trace, sizeof(tr));
    const char* names[9] = {"start", "loaded", "gram", "allreduce", "chol", "inverse+racc", "apply", "cholqr done", "stored"};
    long long ck[2];
    cudaMemcpyFromSymbol(ck, rg::lf_clk, sizeof(ck));
    unsigned long long cnt[3];
    cudaMemcpy(cnt, ws + rg::leaf_stats_offset(), sizeof(cnt), cudaMemcpyDeviceToHost);
    printf("  per launch: fast-Gram fallbacks %.2f, CholQR passes %.2f (%llu launches)\n", cnt[1] / (double)cnt[0], cnt[2] / (double)cnt[0], cnt[0]);
    printf("  gram16: mma %.2f, epilogue %.2f us\n", (tr[25] - tr[1]) / 1e3, (tr[2] - tr[25]) / 1e3);
    printf("  SM clock during the kernel: %.0f MHz\n", (ck[1] - ck[0]) / ((tr[8] - tr[0]) * 1e-3));
    printf("  allreduce: barrier 1 %.2f, reduce %.2f, barrier 2 %.2f, to smem %.2f us\n", (tr[20] - tr[2]) / 1e3,
           (tr[21] - tr[20]) / 1e3, (tr[22] - tr[21]) / 1e3, (tr[3] - tr[22]) / 1e3);
    printf("  chol phase: gdiag / build_g %.2f, check %.2f, factor %.2f, tail %.2f us\n", (tr[26] - tr[3]) / 1e3,
           (tr[27] - tr[26]) / 1e3, (tr[28] - tr[27]) / 1e3, (tr[4] - tr[28]) / 1e3);
    if (L.pq) printf("  prologue: qa load %.2f, k1 %.2f, allreduce %.2f, R_AB %.2f, k2 %.2f us\n", (tr[10] - tr[0]) / 1e3,
                     (tr[11] - tr[10]) / 1e3, (tr[12] - tr[11]) / 1e3, (tr[13] - tr[12]) / 1e3, (tr[1] - tr[13]) / 1e3);
    for (int i = 1; i < 9; ++i) printf("  %-14s %7.2f us (+%.2f)\n", names[i], (tr[i] - tr[0]) / 1e3, ((long long)tr[i] - (long long)tr[i - 1]) / 1e3);
    return 0;
}
