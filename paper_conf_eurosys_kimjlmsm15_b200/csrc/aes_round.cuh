// aes_round.cuh -- AES-128 encryption of one counter block with bank-replicated
// T-tables in shared memory (FIPS-197 §5.1; T-table formulation of
// SubBytes+ShiftRows+MixColumns).  Used by k_aes.cu and k_fused.cu.
//
// Layout: four 1-KB tables T0..T3 (Tj = rotl(T0, 8j) on
// little-endian column words), each replicated 32x so that lane l only ever
// reads bank l: entry x of table j lives at byte
//     (j>>1)*65536 + x*256 + (j&1)*128 + lane*4.
// With that layout one PRMT builds the whole shared address from the state
// word and the lane:  __byte_perm(s, lane*4, 0x5504 | r<<4) = (byte_r(s) << 8) | lane*4,
// so a lookup is PRMT + LDS, bank-conflict free for any data (also removing
// data-dependent shared-memory timing).
#pragma once
#include "internal.cuh"

namespace nba {


// Build the replicated tables from the 1-KB base T0 (global).  All threads of
// the block participate; caller synchronises afterwards.
__device__ __forceinline__ void aes_tables_to_smem(uint8_t *smem, const uint32_t *te0)
{
    uint32_t *tw = reinterpret_cast<uint32_t *>(smem);
    // all base-table loads first (independent), then the replicated stores
    constexpr uint32_t NE = 256u * 32u;
    for (uint32_t e0 = 0; e0 < NE; e0 += 8u * blockDim.x) {
        uint32_t v[8];
#pragma unroll
        for (int u = 0; u < 8; u++) {
            uint32_t e = e0 + threadIdx.x + u * blockDim.x;
            v[u] = e < NE ? __ldg(&te0[e >> 5]) : 0u;
        }
#pragma unroll
        for (int u = 0; u < 8; u++) {
            uint32_t e = e0 + threadIdx.x + u * blockDim.x;
            if (e < NE) {
                uint32_t x = e >> 5, l = e & 31u;
                tw[x * 64u + l] = v[u];
                tw[x * 64u + 32u + l] = __funnelshift_l(v[u], v[u], 8);
                tw[16384u + x * 64u + l] = __funnelshift_l(v[u], v[u], 16);
                tw[16384u + x * 64u + 32u + l] = __funnelshift_l(v[u], v[u], 24);
            }
        }
    }
}

#define NBA_TE(smem, lane4, reg, row, tbl)                                                     \
    (*reinterpret_cast<const uint32_t *>((smem) + __byte_perm((reg), (lane4), 0x5504u | ((row) << 4)) + \
                                         (((tbl) >> 1) * 65536u + ((tbl) & 1u) * 128u)))

// Full 10-round AES-128 on the column words (s0..s3), round keys rk[0..10].
__device__ __forceinline__ uint4 aes128_encrypt_block(const uint8_t *smem, uint32_t lane4,
                                                      const uint4 *rk, uint32_t s0, uint32_t s1,
                                                      uint32_t s2, uint32_t s3)
{
    s0 ^= rk[0].x;
    s1 ^= rk[0].y;
    s2 ^= rk[0].z;
    s3 ^= rk[0].w;
#pragma unroll
    for (int r = 1; r < 10; r++) {
        uint32_t t0 = NBA_TE(smem, lane4, s0, 0, 0) ^ NBA_TE(smem, lane4, s1, 1, 1) ^
                      NBA_TE(smem, lane4, s2, 2, 2) ^ NBA_TE(smem, lane4, s3, 3, 3) ^ rk[r].x;
        uint32_t t1 = NBA_TE(smem, lane4, s1, 0, 0) ^ NBA_TE(smem, lane4, s2, 1, 1) ^
                      NBA_TE(smem, lane4, s3, 2, 2) ^ NBA_TE(smem, lane4, s0, 3, 3) ^ rk[r].y;
        uint32_t t2 = NBA_TE(smem, lane4, s2, 0, 0) ^ NBA_TE(smem, lane4, s3, 1, 1) ^
                      NBA_TE(smem, lane4, s0, 2, 2) ^ NBA_TE(smem, lane4, s1, 3, 3) ^ rk[r].z;
        uint32_t t3 = NBA_TE(smem, lane4, s3, 0, 0) ^ NBA_TE(smem, lane4, s0, 1, 1) ^
                      NBA_TE(smem, lane4, s1, 2, 2) ^ NBA_TE(smem, lane4, s2, 3, 3) ^ rk[r].w;
        s0 = t0;
        s1 = t1;
        s2 = t2;
        s3 = t3;
    }
    // final round: SubBytes + ShiftRows + AddRoundKey; S[x] is byte (j+2)&3 of Tj[x]
    uint4 o;
    o.x = ((NBA_TE(smem, lane4, s0, 0, 2) & 0x000000ffu) | (NBA_TE(smem, lane4, s1, 1, 3) & 0x0000ff00u) |
           (NBA_TE(smem, lane4, s2, 2, 0) & 0x00ff0000u) | (NBA_TE(smem, lane4, s3, 3, 1) & 0xff000000u)) ^ rk[10].x;
    o.y = ((NBA_TE(smem, lane4, s1, 0, 2) & 0x000000ffu) | (NBA_TE(smem, lane4, s2, 1, 3) & 0x0000ff00u) |
           (NBA_TE(smem, lane4, s3, 2, 0) & 0x00ff0000u) | (NBA_TE(smem, lane4, s0, 3, 1) & 0xff000000u)) ^ rk[10].y;
    o.z = ((NBA_TE(smem, lane4, s2, 0, 2) & 0x000000ffu) | (NBA_TE(smem, lane4, s3, 1, 3) & 0x0000ff00u) |
           (NBA_TE(smem, lane4, s0, 2, 0) & 0x00ff0000u) | (NBA_TE(smem, lane4, s1, 3, 1) & 0xff000000u)) ^ rk[10].z;
    o.w = ((NBA_TE(smem, lane4, s3, 0, 2) & 0x000000ffu) | (NBA_TE(smem, lane4, s0, 1, 3) & 0x0000ff00u) |
           (NBA_TE(smem, lane4, s1, 2, 0) & 0x00ff0000u) | (NBA_TE(smem, lane4, s2, 3, 1) & 0xff000000u)) ^ rk[10].w;
    return o;
}

}  // namespace nba
