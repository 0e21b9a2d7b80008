// host_tables.cpp -- setup-time (a0) arithmetic of the library: the AES S-box
// and T-table, AES-128 key schedules and HMAC-SHA1 midstates.
//
// Written independently of oracle/ (which derives its S-box by brute-force
// inversion): here the multiplicative inverse comes from log/antilog tables
// over the generator {03} of GF(2^8)*, FIPS-197 §4.2 / §5.1.1.
//
// PAPER.md:395 (§4.1): "initialize envelope contexts for all flows on startup
// and reuse them by only changing initial vector (IV) values" -> everything
// key-dependent is computed once per SA here, never per packet.
#include <cstdint>
#include <cstring>

#include "internal.cuh"
#include "nba_ipsec.h"

namespace nba {

namespace {

struct AesTables {
    uint8_t sbox[256];
    uint32_t te0[256];   // little-endian column word {2S, S, S, 3S} (row 0 in bits 0..7)
    AesTables()
    {
        // antilog/log over generator 3: alog[i] = 3^i
        uint8_t alog[256], log[256];
        uint8_t v = 1;
        for (int i = 0; i < 255; i++) {
            alog[i] = v;
            log[v] = static_cast<uint8_t>(i);
            // v *= 3  ==  v ^ xtime(v)
            uint8_t x2 = static_cast<uint8_t>((v << 1) ^ ((v & 0x80) ? 0x1b : 0));
            v = static_cast<uint8_t>(v ^ x2);
        }
        alog[255] = 1;
        for (int x = 0; x < 256; x++) {
            uint8_t inv = x ? alog[(255 - log[x]) % 255] : 0;
            // affine map as the matrix form: s = inv ^ rotl(inv,1..4) ^ 0x63
            uint8_t s = inv;
            uint8_t r = inv;
            for (int k = 0; k < 4; k++) {
                r = static_cast<uint8_t>((r << 1) | (r >> 7));
                s ^= r;
            }
            sbox[x] = static_cast<uint8_t>(s ^ 0x63);
        }
        for (int x = 0; x < 256; x++) {
            uint32_t s1 = sbox[x];
            uint32_t s2 = ((s1 << 1) ^ ((s1 & 0x80) ? 0x1b : 0)) & 0xff;
            uint32_t s3 = s2 ^ s1;
            te0[x] = s2 | (s1 << 8) | (s1 << 16) | (s3 << 24);
        }
    }
};

const AesTables &tables()
{
    static const AesTables t;
    return t;
}

inline uint32_t rol(uint32_t x, int n) { return (x << n) | (x >> (32 - n)); }

void sha1_block(uint32_t h[5], const uint8_t blk[64])
{
    uint32_t w[80];
    for (int i = 0; i < 16; i++)
        w[i] = (uint32_t(blk[4 * i]) << 24) | (uint32_t(blk[4 * i + 1]) << 16) |
               (uint32_t(blk[4 * i + 2]) << 8) | uint32_t(blk[4 * i + 3]);
    for (int i = 16; i < 80; i++) w[i] = rol(w[i - 3] ^ w[i - 8] ^ w[i - 14] ^ w[i - 16], 1);
    uint32_t a = h[0], b = h[1], c = h[2], d = h[3], e = h[4];
    static const uint32_t K[4] = {0x5a827999u, 0x6ed9eba1u, 0x8f1bbcdcu, 0xca62c1d6u};
    for (int i = 0; i < 80; i++) {
        uint32_t f = i < 20 ? ((b & c) | (~b & d))
                   : i < 40 ? (b ^ c ^ d)
                   : i < 60 ? ((b & c) | (b & d) | (c & d))
                            : (b ^ c ^ d);
        uint32_t tmp = rol(a, 5) + f + e + K[i / 20] + w[i];
        e = d;
        d = c;
        c = rol(b, 30);
        b = a;
        a = tmp;
    }
    h[0] += a; h[1] += b; h[2] += c; h[3] += d; h[4] += e;
}

}  // namespace

const uint32_t *host_te0() { return tables().te0; }
const uint8_t *host_sbox() { return tables().sbox; }

void aes128_schedule_bytes(const uint8_t key[16], uint8_t rk[176])
{
    const uint8_t *S = tables().sbox;
    std::memcpy(rk, key, 16);
    uint8_t rc = 1;
    for (int i = 16; i < 176; i += 4) {
        uint8_t t0 = rk[i - 4], t1 = rk[i - 3], t2 = rk[i - 2], t3 = rk[i - 1];
        if ((i & 15) == 0) {
            uint8_t u = t0;
            t0 = static_cast<uint8_t>(S[t1] ^ rc);
            t1 = S[t2];
            t2 = S[t3];
            t3 = S[u];
            rc = static_cast<uint8_t>((rc << 1) ^ ((rc & 0x80) ? 0x1b : 0));
        }
        rk[i] = rk[i - 16] ^ t0;
        rk[i + 1] = rk[i - 15] ^ t1;
        rk[i + 2] = rk[i - 14] ^ t2;
        rk[i + 3] = rk[i - 13] ^ t3;
    }
}

void hmac_midstates(const uint8_t key[20], uint32_t hin[5], uint32_t hout[5])
{
    static const uint32_t IV[5] = {0x67452301u, 0xefcdab89u, 0x98badcfeu, 0x10325476u,
                                   0xc3d2e1f0u};
    uint8_t blk[64];
    std::memset(blk, 0, 64);
    std::memcpy(blk, key, 20);
    uint8_t bi[64], bo[64];
    for (int i = 0; i < 64; i++) {
        bi[i] = blk[i] ^ 0x36;
        bo[i] = blk[i] ^ 0x5c;
    }
    std::memcpy(hin, IV, sizeof(IV));
    std::memcpy(hout, IV, sizeof(IV));
    sha1_block(hin, bi);
    sha1_block(hout, bo);
}

}  // namespace nba

extern "C" void nba_ipsec_host_aes128_key_schedule(const uint8_t key[16], uint32_t w[44])
{
    uint8_t rk[176];
    nba::aes128_schedule_bytes(key, rk);
    for (int i = 0; i < 44; i++)
        w[i] = (uint32_t(rk[4 * i]) << 24) | (uint32_t(rk[4 * i + 1]) << 16) |
               (uint32_t(rk[4 * i + 2]) << 8) | uint32_t(rk[4 * i + 3]);
}

extern "C" void nba_ipsec_host_hmac_sha1_midstates(const uint8_t key[20], uint32_t hin[5],
                                                   uint32_t hout[5])
{
    nba::hmac_midstates(key, hin, hout);
}
