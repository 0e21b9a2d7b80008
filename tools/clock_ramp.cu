// Clock / work-rate ramp at the start of an ALU-heavy persistent kernel (GPU).
// Question: does the first ~30 us of a launch that follows an idle GPU (the
// bench's sleep kernel, a host sync) run slower than the steady state?  Each
// CTA (148 x 512 threads, one per SM) runs a dependent integer chain and its
// thread 0 stamps (globaltimer, clock64) every CHUNK iterations; the effective
// SM clock of an interval is d(clock64) / d(globaltimer).  Three cases:
//   idle  : 100 us single-thread sleep kernel, then the ALU kernel
//   warm  : the ALU kernel right after another ALU kernel (no gap)
//   synced: host synchronize, then the ALU kernel
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/clock_ramp tools/clock_ramp.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

constexpr int NST = 64;         // stamps per CTA
constexpr int CHUNK = 256;      // iterations between stamps

__device__ __forceinline__ unsigned long long gtimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void k_spin(long long cycles)
{
    const long long t0 = clock64();
    while (clock64() - t0 < cycles) {}
}

__global__ void __launch_bounds__(512, 1) k_alu(unsigned long long *st, uint32_t *sink)
{
    uint32_t a = threadIdx.x * 0x9e3779b9u, b = blockIdx.x + 1u, c = a ^ 0x5bd1e995u, d = ~a;
    for (int s = 0; s < NST; s++) {
        if (threadIdx.x == 0) {
            st[((size_t)blockIdx.x * NST + s) * 2] = gtimer();
            st[((size_t)blockIdx.x * NST + s) * 2 + 1] = (unsigned long long)clock64();
        }
#pragma unroll 4
        for (int i = 0; i < CHUNK; i++) {   // four independent chains, SHA-1-like mix
            a = __funnelshift_l(a, a, 5) + (b ^ c ^ d) + 0x6ed9eba1u;
            b = __funnelshift_l(b, b, 30) ^ a;
            c = (c + a) ^ __funnelshift_l(d, d, 7);
            d = d + (a & c) + (b | ~d);
        }
    }
    if ((a ^ b ^ c ^ d) == 0x12345678u) sink[0] = a;
}

static void report(const char *name, const std::vector<unsigned long long> &h, int G)
{
    // per interval s: median over CTAs of the effective MHz and of the interval length
    printf("{\"case\": \"%s\", \"intervals\": [", name);
    unsigned long long t00 = ~0ull;
    for (int g = 0; g < G; g++) t00 = std::min(t00, h[((size_t)g * NST) * 2]);
    for (int s = 0; s + 1 < NST; s++) {
        std::vector<double> mhz, ns, at;
        for (int g = 0; g < G; g++) {
            const size_t i = ((size_t)g * NST + s) * 2, j = i + 2;
            const double dt = (double)(h[j] - h[i]), dc = (double)(h[j + 1] - h[i + 1]);
            mhz.push_back(dc / dt * 1e3);
            ns.push_back(dt);
            at.push_back((double)(h[i] - t00));
        }
        std::sort(mhz.begin(), mhz.end());
        std::sort(ns.begin(), ns.end());
        std::sort(at.begin(), at.end());
        printf("%s[%.2f, %.0f, %.0f, %.0f]", s ? ", " : "", at[G / 2] / 1e3, mhz[G / 2], mhz[0],
               ns[G / 2]);
    }
    printf("], \"fields\": \"[start us (median CTA), MHz median, MHz min, interval ns median]\"}\n");
}

int main()
{
    int G = 0;
    cudaDeviceGetAttribute(&G, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long *st;
    uint32_t *sink;
    cudaMalloc(&st, (size_t)G * NST * 2 * sizeof(unsigned long long));
    cudaMalloc(&sink, 4);
    std::vector<unsigned long long> h((size_t)G * NST * 2);
    auto fetch = [&]() {
        cudaDeviceSynchronize();
        cudaMemcpy(h.data(), st, h.size() * 8, cudaMemcpyDeviceToHost);
    };
    for (int w = 0; w < 20; w++) k_alu<<<G, 512>>>(st, sink);   // settle clocks
    cudaDeviceSynchronize();
    for (int rep = 0; rep < 2; rep++) {
        k_spin<<<1, 1>>>(200000);        // ~100 us on one SM, the rest idle
        k_alu<<<G, 512>>>(st, sink);
        fetch();
        report("idle", h, G);
        k_alu<<<G, 512>>>(st, sink);
        k_alu<<<G, 512>>>(st, sink);
        fetch();
        report("warm", h, G);
        cudaDeviceSynchronize();
        k_alu<<<G, 512>>>(st, sink);
        fetch();
        report("synced", h, G);
    }
    printf("{\"err\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
