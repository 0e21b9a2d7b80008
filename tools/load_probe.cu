// Burst-load probe: how long do the fused kernel's per-packet loads take when
// all 148 x 448 lanes issue them at once?  Each variant times (globaltimer,
// per CTA, max over threads) a burst of:
//   sa  : two 256-bit loads of a random SA's 128-byte line (1024 SAs)
//   tos : one byte of the packet's 2 KB pool slot (offset 143)
//   both, and both with the L2 flushed (256 MiB memset) before the kernel.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long gt()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void __launch_bounds__(512, 1)
k_probe(const uint4 *sal, const uint8_t *pool, const uint32_t *sa_idx, int mode, unsigned long long *out,
        uint32_t *sink)
{
    __shared__ unsigned long long t0, t1;
    const uint32_t i = blockIdx.x * 448 + threadIdx.x;
    if (threadIdx.x == 0) { t0 = gt(); t1 = 0; }
    __syncthreads();
    uint32_t acc = 0;
    if (threadIdx.x < 448) {
        const uint32_t s = sa_idx[i];
        if (mode & 1) {
            uint32_t v[8], w[8];
            const uint4 *l = sal + (size_t)s * 8;
            asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                         : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]) : "l"(l));
            asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                         : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7]) : "l"(l + 2));
            for (int k = 0; k < 8; k++) acc ^= v[k] ^ w[k];
        }
        if (mode & 2) acc ^= __ldg(pool + (size_t)i * 2048 + 143);
        if (mode & 4) {   // the 4 coalesced metadata loads
            acc ^= __ldg(sa_idx + i + 65536) ^ __ldg(sa_idx + i + 2 * 65536) ^ __ldg(sa_idx + i + 3 * 65536);
        }
    }
    if (acc == 0x12345678u) sink[0] = acc;
    atomicMax(&t1, gt());
    __syncthreads();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}

__global__ void k_fill(uint4 *p, size_t n)
{
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        p[i] = make_uint4(i, 0, 0, 0);
}

int main()
{
    const int G = 148, N = 448 * G;
    uint4 *sal, *flush;
    uint8_t *pool;
    uint32_t *sa, *sink;
    unsigned long long *out;
    cudaMalloc(&sal, 1024 * 128);
    cudaMalloc(&pool, (size_t)N * 2048);
    cudaMalloc(&sa, (size_t)N * 4 * 4);
    cudaMalloc(&sink, 64);
    cudaMalloc(&out, G * 8);
    const size_t nf = (256u << 20) / 16;
    cudaMalloc(&flush, nf * 16);
    uint32_t *h = new uint32_t[N * 4];
    uint32_t x = 12345;
    for (int k = 0; k < N * 4; k++) { x = x * 1664525u + 1013904223u; h[k] = (x >> 8) % 1024; }
    cudaMemcpy(sa, h, (size_t)N * 16, cudaMemcpyHostToDevice);
    cudaMemset(sal, 1, 1024 * 128);
    cudaMemset(pool, 2, (size_t)N * 2048);
    unsigned long long ho[G];
    const char *names[] = {"", "sa", "tos", "sa+tos", "meta", "sa+meta", "tos+meta", "sa+tos+meta"};
    printf("{\n");
    for (int fl = 0; fl < 2; fl++)
        for (int mode = 1; mode < 8; mode++) {
            double best = 1e30, med = 0;
            for (int rep = 0; rep < 5; rep++) {
                if (fl) k_fill<<<G * 4, 512>>>(flush, nf);
                k_probe<<<G, 512>>>(sal, pool, sa, mode, out, sink);
                cudaDeviceSynchronize();
                cudaMemcpy(ho, out, sizeof(ho), cudaMemcpyDeviceToHost);
                unsigned long long mx = 0, sum = 0;
                for (int c = 0; c < G; c++) { mx = ho[c] > mx ? ho[c] : mx; sum += ho[c]; }
                if (mx < best) { best = mx; med = (double)sum / G; }
            }
            printf("  \"%s%s\": {\"max_us\": %.2f, \"mean_us\": %.2f},\n", names[mode], fl ? "_flushed" : "", best / 1e3, med / 1e3);
        }
    printf("  \"done\": 1\n}\n");
    return 0;
}
