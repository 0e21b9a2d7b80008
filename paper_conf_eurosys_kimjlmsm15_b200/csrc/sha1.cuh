// sha1.cuh -- SHA-1 compression (FIPS 180-4 §6.1.2) with the 16-word message
// schedule kept in registers as a circular buffer, for HMAC-SHA1-96
// (RFC 2104 / RFC 2404).  Used by k_hmac.cu and k_fused.cu.
#pragma once
#include "internal.cuh"

namespace nba {

__device__ __forceinline__ uint32_t rotl32(uint32_t x, int n) { return __funnelshift_l(x, x, n); }

// st[5] <- compress(st, w[16]); w is clobbered (holds W[64..79]).
__device__ __forceinline__ void sha1_compress(uint32_t st[5], uint32_t w[16])
{
    uint32_t a = st[0], b = st[1], c = st[2], d = st[3], e = st[4];
#pragma unroll
    for (int t = 0; t < 80; t++) {
        uint32_t wt;
        if (t < 16) {
            wt = w[t];
        } else {
            wt = rotl32(w[(t - 3) & 15] ^ w[(t - 8) & 15] ^ w[(t - 14) & 15] ^ w[t & 15], 1);
            w[t & 15] = wt;
        }
        uint32_t f, k;
        if (t < 20) {
            f = (b & c) | (~b & d);
            k = 0x5a827999u;
        } else if (t < 40) {
            f = b ^ c ^ d;
            k = 0x6ed9eba1u;
        } else if (t < 60) {
            f = (b & c) | (d & (b | c));
            k = 0x8f1bbcdcu;
        } else {
            f = b ^ c ^ d;
            k = 0xca62c1d6u;
        }
        uint32_t tmp = rotl32(a, 5) + f + e + k + wt;
        e = d;
        d = c;
        c = rotl32(b, 30);
        b = a;
        a = tmp;
    }
    st[0] += a;
    st[1] += b;
    st[2] += c;
    st[3] += d;
    st[4] += e;
}

// Same compression with two of each round's additions (e + K + W) issued as
// IMAD on the FMA pipe instead of on the ALU pipe, which the rounds saturate
// (FMA is otherwise idle in the lane loop): -2% / -1% step time at 64 / 1514 B.
// Moving the rotations there too (IMAD.HI + IMAD) or the final addition was
// measured slower.  `one` must be 1 at run time but opaque to the compiler
// (otherwise x * 1 + y folds back into an ALU add).
__device__ __forceinline__ uint32_t mad_u32(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}

__device__ __forceinline__ void sha1_compress_fma(uint32_t st[5], uint32_t w[16], uint32_t one)
{
    uint32_t a = st[0], b = st[1], c = st[2], d = st[3], e = st[4];
#pragma unroll
    for (int t = 0; t < 80; t++) {
        uint32_t wt;
        if (t < 16) {
            wt = w[t];
        } else {
            wt = rotl32(w[(t - 3) & 15] ^ w[(t - 8) & 15] ^ w[(t - 14) & 15] ^ w[t & 15], 1);
            w[t & 15] = wt;
        }
        uint32_t f, k;
        if (t < 20) {
            f = (b & c) | (~b & d);
            k = 0x5a827999u;
        } else if (t < 40) {
            f = b ^ c ^ d;
            k = 0x6ed9eba1u;
        } else if (t < 60) {
            f = (b & c) | (d & (b | c));
            k = 0x8f1bbcdcu;
        } else {
            f = b ^ c ^ d;
            k = 0xca62c1d6u;
        }
        const uint32_t ekw = mad_u32(wt, one, mad_u32(e, one, k));   // e + K + W (FMA pipe)
        const uint32_t tmp = rotl32(a, 5) + f + ekw;                 // IADD3 (ALU)
        e = d;
        d = c;
        c = rotl32(b, 30);
        b = a;
        a = tmp;
    }
    st[0] += a;
    st[1] += b;
    st[2] += c;
    st[3] += d;
    st[4] += e;
}

// Load 16 big-endian message words from a 16-B aligned little-endian image.
__device__ __forceinline__ void sha1_load_block(uint32_t w[16], const uint4 *p)
{
#pragma unroll
    for (int j = 0; j < 4; j++) {
        uint4 v = p[j];
        w[4 * j + 0] = bswap32(v.x);
        w[4 * j + 1] = bswap32(v.y);
        w[4 * j + 2] = bswap32(v.z);
        w[4 * j + 3] = bswap32(v.w);
    }
}

// HMAC-SHA1 of the ESP message M = record[0, 16+C) (SPI..trailer) given the
// SA's inner / outer midstates; returns the first three digest words (ICV).
// `rec` is the 16-B aligned record; reads may extend up to 64 bytes past
// 16+C (the datablock has slack), trailing bytes are masked.
template <typename LoadFn>
__device__ __forceinline__ void hmac_sha1_96(const uint32_t hin[5], const uint32_t hout[5],
                                             uint32_t C, LoadFn load_block, uint32_t icv[3])
{
    const uint32_t M = 16u + C;               // bytes; multiple of 4 (C = 0 mod 4)
    const uint32_t nfull = M >> 6;
    const uint32_t remw = (M & 63u) >> 2;     // words in the last partial block
    const uint32_t nblocks = (M + 8u) / 64u + 1u;
    const uint32_t bitlen = (64u + M) * 8u;   // the ipad block counts in the length
    uint32_t st[5] = {hin[0], hin[1], hin[2], hin[3], hin[4]};
    uint32_t w[16];
    // blocks 0..nblocks-1: inner hash; block nblocks: outer hash of the inner
    // digest (one SHA-1 compression body for both keeps the code compact)
    for (uint32_t b = 0; b <= nblocks; b++) {
        if (b < nblocks) {
            if (b <= nfull) load_block(w, b);
            if (b >= nfull) {                 // FIPS 180-4 §5.1.1 padding
                const uint32_t cut = (b == nfull) ? remw : 0u;
#pragma unroll
                for (uint32_t j = 0; j < 16; j++)
                    w[j] = j < cut ? w[j] : ((b == nfull && j == cut) ? 0x80000000u : 0u);
                if (b == nblocks - 1u) w[15] = bitlen;
            }
        } else {
#pragma unroll
            for (int j = 0; j < 5; j++) {
                w[j] = st[j];
                st[j] = hout[j];
            }
            w[5] = 0x80000000u;
#pragma unroll
            for (int j = 6; j < 15; j++) w[j] = 0u;
            w[15] = (64u + 20u) * 8u;
        }
        sha1_compress(st, w);
    }
    icv[0] = st[0];
    icv[1] = st[1];
    icv[2] = st[2];
}

}  // namespace nba
