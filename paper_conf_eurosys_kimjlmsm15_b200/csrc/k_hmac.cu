// k_hmac.cu -- row a4 of the hot path (unfused pipeline): HMAC-SHA1-96 over
// SPI || seq || IV || ciphertext of every record (encrypt-then-MAC,
// RFC 4303 §3.3.2-§3.3.4; ICV = first 96 bits, RFC 2404), written at
// record[16+C, 16+C+12).
//
// PAPER.md:389 (§4.1): "IPsec encryption uses HMAC-SHA1 to authenticate the
// packets"; this was the dominant kernel on the GTX 680
// (~100 of ~140 us).  SHA-1 is a serial chain per message, so the mapping is
// one lane per packet (32 packets per warp, reading H5 of DESIGN.md), with the
// 16-word schedule in registers and the inner/outer key blocks replaced by
// per-SA midstates computed once at setup (RFC 2104 §4 note on precomputation).
// Packets are visited in W.perm order, which the prologue sorts by SHA-1
// block count so that lanes of a warp do equal work under mixed lengths.
#include "sha1.cuh"

namespace nba {

constexpr int HMAC_THREADS = 128;

__global__ void __launch_bounds__(HMAC_THREADS)
k_hmac(DevTable T, DevWork W, BatchArgs B)
{
    const uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x;
    if (idx >= B.n) return;
    const uint32_t pkt = W.perm[idx];
    const uint32_t info = W.m_info[pkt];
    if (!(info & INFO_OK)) return;
    const uint32_t C = info & 0xffffu;
    const uint32_t sa = B.sa_idx[pkt];
    uint4 *rec = W.db + W.m_rec[pkt];
    const uint4 h0 = __ldg(&T.hmid[(size_t)sa * 3 + 0]);
    const uint4 h1 = __ldg(&T.hmid[(size_t)sa * 3 + 1]);
    const uint4 h2 = __ldg(&T.hmid[(size_t)sa * 3 + 2]);
    const uint32_t hin[5] = {h0.x, h0.y, h0.z, h0.w, h1.x};
    const uint32_t hout[5] = {h1.y, h1.z, h1.w, h2.x, h2.y};
    uint32_t icv[3];
    hmac_sha1_96(hin, hout, C,
                 [&](uint32_t w[16], uint32_t b) { sha1_load_block(w, rec + 4u * b); }, icv);
    uint32_t *dst = reinterpret_cast<uint32_t *>(rec) + ((16u + C) >> 2);
    dst[0] = bswap32(icv[0]);
    dst[1] = bswap32(icv[1]);
    dst[2] = bswap32(icv[2]);
}

cudaError_t launch_hmac(const DevTable &T, const DevWork &W, const BatchArgs &B,
                        cudaStream_t st)
{
    uint32_t grid = (B.n + HMAC_THREADS - 1) / HMAC_THREADS;
    k_hmac<<<grid, HMAC_THREADS, 0, st>>>(T, W, B);
    return cudaGetLastError();
}

}  // namespace nba
