// Instruction-fetch cost of straight-line code at the start of a launch (GPU).
// The pipelined ring's first iteration runs its lane code ~2x slower than the
// next ones, every segment alike and every lane alike (tools/ring_ab.py trace,
// lane timelines): the signature of all warps waiting on the same instruction
// fetches.  This probe measures it on synthetic code: four distinct chunks of
// straight-line integer code (~CHUNK_OPS instructions each), timed per chunk
// with clock64 by every warp of one CTA per SM, in two passes within a launch,
// launched twice back to back:
//   seq : every warp runs chunks 0,1,2,3 (the ring's lanes: all warps in step)
//   par : warp w first runs chunk w % 4 alone (a warm-up split over warps),
//         then chunks 0..3
// Output per mode and launch: median cycles of each chunk in pass 1 / pass 2.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/icache_probe tools/icache_probe.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

#ifndef CHUNK_OPS
#define CHUNK_OPS 640      // ~10 KB of SASS per chunk (16 B per instruction)
#endif

template <int C>
__device__ __noinline__ uint32_t chunk(uint32_t a, uint32_t b)
{
#pragma unroll
    for (int i = 0; i < CHUNK_OPS / 2; i++) {
        a = __funnelshift_l(a, b, (i * 7 + C) & 31) ^ (0x9e3779b9u * (uint32_t)(i + 1 + 1000 * C));
        b = b + (a ^ (0x85ebca6bu + (uint32_t)(i * 13 + C)));
    }
    return a ^ b;
}

__device__ __forceinline__ uint32_t run_chunk(int c, uint32_t a, uint32_t b)
{
    switch (c) {
    case 0: return chunk<0>(a, b);
    case 1: return chunk<1>(a, b);
    case 2: return chunk<2>(a, b);
    default: return chunk<3>(a, b);
    }
}

// out[cta][warp][pass][chunk] cycles (lane 0); mode 0 = seq, 1 = par (pre-pass)
__global__ void __launch_bounds__(512, 1) k_probe(int mode, long long *out, uint32_t *sink)
{
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t a = threadIdx.x * 0x27d4eb2du, b = blockIdx.x + 7u;
    long long pre = 0;
    if (mode == 1) {
        const long long t0 = clock64();
        a ^= run_chunk(warp & 3, a, b);
        pre = clock64() - t0;
        __syncthreads();
    }
    for (int pass = 0; pass < 2; pass++) {
        for (int c = 0; c < 4; c++) {
            const long long t0 = clock64();
            a ^= run_chunk(c, a, b);
            const long long t1 = clock64();
            if (lane == 0) out[(((size_t)blockIdx.x * 16 + warp) * 2 + pass) * 5 + c] = t1 - t0;
        }
        __syncthreads();
    }
    if (lane == 0) out[(((size_t)blockIdx.x * 16 + warp) * 2 + 0) * 5 + 4] = pre;
    if (a == 0x1234567u) sink[0] = b;
}

int main()
{
    int G = 0;
    cudaDeviceGetAttribute(&G, cudaDevAttrMultiProcessorCount, 0);
    long long *out;
    uint32_t *sink;
    const size_t n = (size_t)G * 16 * 2 * 5;
    cudaMalloc(&out, n * 8);
    cudaMalloc(&sink, 4);
    std::vector<long long> h(n);
    for (int w = 0; w < 3; w++) k_probe<<<G, 512>>>(0, out, sink);
    cudaDeviceSynchronize();
    for (int mode = 0; mode < 2; mode++) {
        for (int launch = 0; launch < 3; launch++) {
            k_probe<<<G, 512>>>(mode, out, sink);
            cudaDeviceSynchronize();
            cudaMemcpy(h.data(), out, n * 8, cudaMemcpyDeviceToHost);
            printf("{\"mode\": \"%s\", \"launch\": %d", mode ? "par" : "seq", launch);
            for (int pass = 0; pass < 2; pass++) {
                printf(", \"pass%d\": [", pass + 1);
                for (int c = 0; c < 4; c++) {
                    std::vector<long long> v;
                    for (int g = 0; g < G; g++)
                        for (int w = 0; w < 16; w++) v.push_back(h[(((size_t)g * 16 + w) * 2 + pass) * 5 + c]);
                    std::sort(v.begin(), v.end());
                    printf("%s%lld", c ? ", " : "", v[v.size() / 2]);
                }
                printf("]");
            }
            std::vector<long long> v;
            for (int g = 0; g < G; g++)
                for (int w = 0; w < 16; w++) v.push_back(h[(((size_t)g * 16 + w) * 2) * 5 + 4]);
            std::sort(v.begin(), v.end());
            printf(", \"pre\": %lld}\n", v[v.size() / 2]);
        }
    }
    printf("{\"err\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
