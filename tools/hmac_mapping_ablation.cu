// HMAC-SHA1 work mapping ablation (north_star's "one warp per
// packet"): the same SHA-1 compressions (FIPS 180-4 §6.1.2, the library's
// sha1_compress) for 65,536 messages of 3 compressions each (a 64-B frame's
// HMAC with precomputed midstates), mapped
//   lane : one lane per message (the library's mapping), 512-thread CTAs;
//   warp : one warp per message, lane 0 running the rounds -- SHA-1's rounds
//          are one dependent chain, so the other 31 lanes have nothing to do
//          (the schedule admits at most 3 parallel words per step);
// timed with CUDA events over 20 repetitions after warm-up, output checked
// equal between the two.  Prints compressions per second per mapping.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//        -I paper_conf_eurosys_kimjlmsm15_b200/csrc -I include -o build/hmac_mapping tools/hmac_mapping_ablation.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>
#include "sha1.cuh"

using namespace nba;

constexpr uint32_t N_MSG = 65536, N_COMP = 3;

__device__ __forceinline__ void msg_block(uint32_t m, uint32_t k, uint32_t w[16])
{
#pragma unroll
    for (int j = 0; j < 16; j++) w[j] = m * 0x9E3779B9u + k * 0x85EBCA6Bu + (uint32_t)j * 0xC2B2AE35u;
}

__global__ void __launch_bounds__(512) k_lane(uint32_t *out)
{
    const uint32_t m = blockIdx.x * blockDim.x + threadIdx.x;
    if (m >= N_MSG) return;
    uint32_t st[5] = {0x67452301u, 0xEFCDAB89u, 0x98BADCFEu, 0x10325476u, 0xC3D2E1F0u + m};
    for (uint32_t k = 0; k < N_COMP; k++) {
        uint32_t w[16];
        msg_block(m, k, w);
        sha1_compress(st, w);
    }
    out[m] = st[0] ^ st[1] ^ st[2] ^ st[3] ^ st[4];
}

__global__ void __launch_bounds__(512) k_warp(uint32_t *out)
{
    const uint32_t m = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (m >= N_MSG || (threadIdx.x & 31u) != 0u) return;   // lane 0 of the message's warp
    uint32_t st[5] = {0x67452301u, 0xEFCDAB89u, 0x98BADCFEu, 0x10325476u, 0xC3D2E1F0u + m};
    for (uint32_t k = 0; k < N_COMP; k++) {
        uint32_t w[16];
        msg_block(m, k, w);
        sha1_compress(st, w);
    }
    out[m] = st[0] ^ st[1] ^ st[2] ^ st[3] ^ st[4];
}

int main()
{
    uint32_t *a, *b;
    cudaMalloc(&a, N_MSG * 4);
    cudaMalloc(&b, N_MSG * 4);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int reps = 20;
    float ms_lane = 0, ms_warp = 0;
    for (int w = 0; w < 3; w++) {
        k_lane<<<N_MSG / 512, 512>>>(a);
        k_warp<<<N_MSG * 32 / 512, 512>>>(b);
    }
    cudaEventRecord(e0);
    for (int r = 0; r < reps; r++) k_lane<<<N_MSG / 512, 512>>>(a);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms_lane, e0, e1);
    cudaEventRecord(e0);
    for (int r = 0; r < reps; r++) k_warp<<<N_MSG * 32 / 512, 512>>>(b);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms_warp, e0, e1);
    std::vector<uint32_t> ha(N_MSG), hb(N_MSG);
    cudaMemcpy(ha.data(), a, N_MSG * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(hb.data(), b, N_MSG * 4, cudaMemcpyDeviceToHost);
    bool same = ha == hb;
    const double comps = (double)N_MSG * N_COMP * reps;
    printf("{\"messages\": %u, \"compressions_per_message\": %u, \"same_output\": %s, "
           "\"lane_per_message\": {\"us_per_batch\": %.2f, \"Gcompressions_per_s\": %.2f}, "
           "\"warp_per_message\": {\"us_per_batch\": %.2f, \"Gcompressions_per_s\": %.2f}, "
           "\"ratio\": %.1f, \"err\": \"%s\"}\n",
           N_MSG, N_COMP, same ? "true" : "false", 1e3 * ms_lane / reps, comps / (ms_lane * 1e-3) / 1e9,
           1e3 * ms_warp / reps, comps / (ms_warp * 1e-3) / 1e9, ms_warp / ms_lane,
           cudaGetErrorString(cudaGetLastError()));
    return 0;
}
