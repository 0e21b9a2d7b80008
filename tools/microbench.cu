// microbench.cu -- measured integer / shared-memory peaks of the B200 SM for
// the roofline of the ESP path (SURVEY §8(d) "must be microbenchmarked").
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_eurosys_kimjlmsm15_b200/csrc \
//        -o build/microbench tools/microbench.cu && build/microbench
//
// Prints one JSON object: per-SM-per-clock rates (from clock64 inside the
// kernel) and chip-wide rates (CUDA events) for
//   lds32      conflict-free 32-bit shared loads, index from the previous value
//              with ~3 ALU ops of address arithmetic per load (ALU-bound: kept
//              for comparison with round 1)
//   lds32_prmt the lane loop's T-table pattern: one PRMT + one LDS per lookup
//   lds32_pure loads with fixed addresses (0.5 ALU op per load): the LDS rate
//   lop3/prmt/shf/iadd3   ALU-pipe integer ops
//   aes_block  full T-table AES-128 blocks (aes_round.cuh), no global memory
//   sha1_comp  SHA-1 compressions (sha1.cuh), no global memory
#include <cstdio>
#include <cuda_runtime.h>

#include "aes_round.cuh"
#include "sha1.cuh"

using namespace nba;

#define CK(x)                                                                       \
    do {                                                                            \
        cudaError_t e_ = (x);                                                       \
        if (e_ != cudaSuccess) {                                                    \
            fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e_));                \
            return 1;                                                               \
        }                                                                           \
    } while (0)

constexpr int ITERS = 4096;

__global__ void k_lds(uint32_t *out, unsigned long long *cyc, uint32_t seed)
{
    __shared__ uint32_t t[256 * 32];
    for (int i = threadIdx.x; i < 256 * 32; i += blockDim.x) t[i] = i * 2654435761u;
    __syncthreads();
    uint32_t lane = threadIdx.x & 31;
    uint32_t a0 = seed + threadIdx.x, a1 = a0 * 3, a2 = a0 * 5, a3 = a0 * 7;
    unsigned long long c0 = clock64();
#pragma unroll 4
    for (int i = 0; i < ITERS; i++) {
        // 4 independent dependent chains: index from the previous value (like AES)
        a0 = t[((a0 & 255u) << 5) | lane];
        a1 = t[((a1 & 255u) << 5) | lane];
        a2 = t[((a2 & 255u) << 5) | lane];
        a3 = t[((a3 & 255u) << 5) | lane];
    }
    unsigned long long c1 = clock64();
    if (threadIdx.x == 0) atomicMax(cyc, c1 - c0);
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 ^ a1 ^ a2 ^ a3;
}

// The T-table access pattern of the lane loop (fused_common.cuh TL): a 64 KB
// table image at a 64 KB-aligned shared address, one PRMT forms the whole
// address (byte 0 of the state word -> bits 8..15, lane*4 -> bits 0..7, the
// base -> bits 16..31): 1 ALU op per LDS, 8 independent chains per thread.
__global__ void __launch_bounds__(512, 1) k_lds_prmt(uint32_t *out, unsigned long long *cyc, uint32_t seed)
{
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t sb = (uint32_t)__cvta_generic_to_shared(smem);
    const uint32_t toff = (0x10000u - (sb & 0xffffu)) & 0xffffu;
    uint32_t *tw = reinterpret_cast<uint32_t *>(smem + toff);
    for (uint32_t i = threadIdx.x; i < 16384u; i += blockDim.x) tw[i] = (i * 2654435761u) ^ seed;
    __syncthreads();
    const uint32_t lane4r = ((threadIdx.x & 31u) * 4u) | ((sb + toff) & 0xffff0000u);
    uint32_t a[8];
#pragma unroll
    for (int k = 0; k < 8; k++) a[k] = seed * (threadIdx.x + 1u) + 977u * k;
    unsigned long long c0 = clock64();
#pragma unroll 2
    for (int i = 0; i < ITERS; i++) {
#pragma unroll
        for (int k = 0; k < 8; k++) {
            const uint32_t ad = __byte_perm(a[k], lane4r, 0x7604u | ((k & 3) << 4));
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(a[k]) : "r"(ad));
        }
    }
    unsigned long long c1 = clock64();
    if (threadIdx.x == 0) atomicMax(cyc, c1 - c0);
    uint32_t x = 0;
#pragma unroll
    for (int k = 0; k < 8; k++) x ^= a[k];
    out[blockIdx.x * blockDim.x + threadIdx.x] = x;
}

// Shared-memory loads with no address arithmetic (fixed per-lane addresses,
// conflict-free, volatile so they are not hoisted): 16 loads and 8 three-input
// XORs per iteration -- the LDS rate with the ALU pipe nearly idle.
__global__ void __launch_bounds__(512, 1) k_lds_pure(uint32_t *out, unsigned long long *cyc, uint32_t seed)
{
    __shared__ uint32_t t[16 * 32 * 8];
    for (uint32_t i = threadIdx.x; i < 16u * 32u * 8u; i += blockDim.x) t[i] = i * 2654435761u ^ seed;
    __syncthreads();
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(&t[(threadIdx.x & 31u) + 512u * ((threadIdx.x >> 5) & 7u)]);
    uint32_t acc0 = 0, acc1 = 0;
    unsigned long long c0 = clock64();
#pragma unroll 1
    for (int i = 0; i < ITERS; i++) {
        uint32_t v[16];
#define LDK(k) asm volatile("ld.shared.u32 %0, [%1+" #k "];" : "=r"(v[(k) / 128]) : "r"(base))
        LDK(0); LDK(128); LDK(256); LDK(384); LDK(512); LDK(640); LDK(768); LDK(896);
        LDK(1024); LDK(1152); LDK(1280); LDK(1408); LDK(1536); LDK(1664); LDK(1792); LDK(1920);
#undef LDK
#pragma unroll
        for (int k = 0; k < 16; k += 4) {
            acc0 ^= v[k] ^ v[k + 1];
            acc1 ^= v[k + 2] ^ v[k + 3];
        }
    }
    unsigned long long c1 = clock64();
    if (threadIdx.x == 0) atomicMax(cyc, c1 - c0);
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc0 ^ acc1;
}

template <int OP>
__global__ void k_alu(uint32_t *out, unsigned long long *cyc, uint32_t seed)
{
    uint32_t r[8];
#pragma unroll
    for (int j = 0; j < 8; j++) r[j] = seed * (threadIdx.x + 1) + j;
    unsigned long long c0 = clock64();
#pragma unroll 4
    for (int i = 0; i < ITERS; i++) {
#pragma unroll
        for (int j = 0; j < 8; j++) {
            if (OP == 0) r[j] = (r[j] ^ r[(j + 1) & 7]) & r[(j + 3) & 7];             // LOP3
            if (OP == 1) r[j] = __byte_perm(r[j], r[(j + 1) & 7], 0x5140 + j);        // PRMT
            if (OP == 2) r[j] = __funnelshift_l(r[j], r[j], 5 + j);                   // SHF
            if (OP == 3) r[j] = r[j] + r[(j + 1) & 7] + r[(j + 5) & 7];               // IADD3
        }
    }
    unsigned long long c1 = clock64();
    if (threadIdx.x == 0) atomicMax(cyc, c1 - c0);
    uint32_t x = 0;
#pragma unroll
    for (int j = 0; j < 8; j++) x ^= r[j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = x;
}

constexpr int AES_ITERS = 64;

__global__ void __launch_bounds__(512, 1) k_aesonly(uint32_t *out, unsigned long long *cyc,
                                                      const uint32_t *te0, const uint4 *rkg)
{
    extern __shared__ __align__(16) uint8_t smem[];
    aes_tables_to_smem(smem, te0);
    __syncthreads();
    uint4 rk[11];
#pragma unroll
    for (int r = 0; r < 11; r++) rk[r] = rkg[r];
    const uint32_t lane4 = (threadIdx.x & 31) * 4;
    uint32_t s0 = threadIdx.x, s1 = blockIdx.x, s2 = 7, s3 = 9;
    unsigned long long c0 = clock64();
    for (int i = 0; i < AES_ITERS; i++) {
        uint4 o = aes128_encrypt_block(smem, lane4, rk, s0, s1, s2, s3 + i);
        s0 ^= o.x;
        s1 ^= o.y;
        s2 ^= o.z;
        s3 ^= o.w;
    }
    unsigned long long c1 = clock64();
    if (threadIdx.x == 0) atomicMax(cyc, c1 - c0);
    out[blockIdx.x * blockDim.x + threadIdx.x] = s0 ^ s1 ^ s2 ^ s3;
}

constexpr int SHA_ITERS = 64;

__global__ void k_shaonly(uint32_t *out, unsigned long long *cyc, uint32_t seed)
{
    uint32_t st[5] = {seed, seed * 3, seed * 5, seed * 7, threadIdx.x};
    uint32_t w[16];
#pragma unroll
    for (int j = 0; j < 16; j++) w[j] = seed ^ (threadIdx.x * 16 + j);
    unsigned long long c0 = clock64();
    for (int i = 0; i < SHA_ITERS; i++) {
        sha1_compress(st, w);
        w[0] ^= st[0];
    }
    unsigned long long c1 = clock64();
    if (threadIdx.x == 0) atomicMax(cyc, c1 - c0);
    out[blockIdx.x * blockDim.x + threadIdx.x] = st[0] ^ st[1] ^ st[2] ^ st[3] ^ st[4];
}

int main()
{
    int dev = 0, nsm = 0, clk_khz = 0;
    CK(cudaSetDevice(dev));
    CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
    CK(cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev));
    uint32_t *out;
    unsigned long long *cyc;
    CK(cudaMalloc(&out, 64u << 20));
    CK(cudaMalloc(&cyc, 8));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto run = [&](auto launch, double ops_per_thread, int blocks, int threads, const char *name,
                   bool last) -> int {
        for (int w = 0; w < 3; w++) launch();           // warm up clocks
        CK(cudaMemset(cyc, 0, 8));
        cudaEventRecord(e0);
        launch();
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        unsigned long long c = 0;
        CK(cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost));
        double total = ops_per_thread * blocks * threads;
        double per_sm_clk = ops_per_thread * threads * ((double)blocks / nsm) / (double)c;
        printf("  \"%s\": {\"per_sm_per_clk\": %.3f, \"chip_G_per_s\": %.2f, \"ms\": %.4f, "
               "\"blocks\": %d, \"threads\": %d}%s\n",
               name, per_sm_clk, total / (ms * 1e-3) / 1e9, ms, blocks, threads, last ? "" : ",");
        return 0;
    };
    printf("{\n  \"sms\": %d, \"clock_khz_attr\": %d,\n", nsm, clk_khz);
    const int B = nsm * 2, TH = 1024;
    run([&] { k_lds<<<B, TH>>>(out, cyc, 1); }, 4.0 * ITERS, B, TH, "lds32_lanes", false);
    CK(cudaFuncSetAttribute(k_lds_prmt, cudaFuncAttributeMaxDynamicSharedMemorySize, 131072));
    run([&] { k_lds_prmt<<<nsm, 512, 131072>>>(out, cyc, 1); }, 8.0 * ITERS, nsm, 512,
        "lds32_prmt_lanes", false);
    run([&] { k_lds_pure<<<nsm, 512>>>(out, cyc, 1); }, 16.0 * ITERS, nsm, 512, "lds32_pure_lanes",
        false);
    run([&] { k_lds_pure<<<nsm * 2, 512>>>(out, cyc, 1); }, 16.0 * ITERS, nsm * 2, 512,
        "lds32_pure_lanes_2cta", false);
    run([&] { k_alu<0><<<B, TH>>>(out, cyc, 1); }, 8.0 * ITERS, B, TH, "lop3_lanes", false);
    run([&] { k_alu<1><<<B, TH>>>(out, cyc, 1); }, 8.0 * ITERS, B, TH, "prmt_lanes", false);
    run([&] { k_alu<2><<<B, TH>>>(out, cyc, 1); }, 8.0 * ITERS, B, TH, "shf_lanes", false);
    run([&] { k_alu<3><<<B, TH>>>(out, cyc, 1); }, 8.0 * ITERS, B, TH, "iadd3_lanes", false);
    // AES: real tables
    uint32_t te0_h[256];
    {
        uint8_t sb[256], alog[256], lg[256];
        uint8_t v = 1;
        for (int i = 0; i < 255; i++) {
            alog[i] = v;
            lg[v] = (uint8_t)i;
            uint8_t x2 = (uint8_t)((v << 1) ^ ((v & 0x80) ? 0x1b : 0));
            v = (uint8_t)(v ^ x2);
        }
        for (int x = 0; x < 256; x++) {
            uint8_t inv = x ? alog[(255 - lg[x]) % 255] : 0, s = inv, r = inv;
            for (int k = 0; k < 4; k++) {
                r = (uint8_t)((r << 1) | (r >> 7));
                s ^= r;
            }
            sb[x] = (uint8_t)(s ^ 0x63);
        }
        for (int x = 0; x < 256; x++) {
            uint32_t s1 = sb[x], s2 = ((s1 << 1) ^ ((s1 & 0x80) ? 0x1b : 0)) & 0xff;
            te0_h[x] = s2 | (s1 << 8) | (s1 << 16) | ((s2 ^ s1) << 24);
        }
    }
    uint32_t *te0;
    uint4 *rk;
    CK(cudaMalloc(&te0, 1024));
    CK(cudaMalloc(&rk, 176));
    CK(cudaMemcpy(te0, te0_h, 1024, cudaMemcpyHostToDevice));
    CK(cudaMemset(rk, 0x5a, 176));
    CK(cudaFuncSetAttribute(k_aesonly, cudaFuncAttributeMaxDynamicSharedMemorySize, 131072));
    for (int th : {256, 512}) {
        char nm[64];
        snprintf(nm, sizeof nm, "aes_block_t%d", th);
        run([&] { k_aesonly<<<nsm, th, 131072>>>(out, cyc, te0, rk); }, (double)AES_ITERS, nsm, th,
            nm, false);
    }
    run([&] { k_shaonly<<<B, 512>>>(out, cyc, 1); }, (double)SHA_ITERS, B, 512, "sha1_comp_t512x2",
        false);
    run([&] { k_shaonly<<<nsm, 512>>>(out, cyc, 1); }, (double)SHA_ITERS, nsm, 512,
        "sha1_comp_t512x1", false);
    run([&] { k_shaonly<<<nsm, 256>>>(out, cyc, 1); }, (double)SHA_ITERS, nsm, 256,
        "sha1_comp_t256x1", true);
    printf("}\n");
    return 0;
}
