// k_scatter.cu -- row a5 of the hot path (unfused pipeline): write each
// finished ESP packet to its caller-provided output slot:
//     outer IPv4 header (20 B) || record[0, 28+C)      -> out_buf + out_off[i]
// and out_len[i] = 48 + C (0 when dropped), and accumulate device counters.
//
// Outer header (reading A13; RFC 4301 §5.1.2.1, RFC 791, RFC 1071):
//   45 | TOS copied from the inner header | BE16(48+C) | ID 0 | DF | TTL 64 |
//   proto 50 (ESP) | checksum | tunnel src | tunnel dst.
// PAPER.md:327 / :343 (§3.3): the offload's postprocessing writes results back
// into the packets ("whole pkt" datablocks with a size delta, Table 2).
//
// One CTA per 1024-packet tile; each thread writes 16-byte chunks aligned to
// the DESTINATION address (full chunks are one st.global.v4; the unaligned
// head/tail chunks are written byte by byte so no byte outside
// [out_off, out_off + out_len) is touched).
#include "internal.cuh"

namespace nba {

__device__ __forceinline__ void outer_header_words(uint32_t tos, uint32_t L, uint32_t src_img,
                                                   uint32_t dst_img, uint32_t hw[5])
{
    uint32_t src = bswap32(src_img), dst = bswap32(dst_img);
    uint32_t sum = (0x4500u | tos) + L + 0x4000u + ((64u << 8) | 50u) + (src >> 16) +
                   (src & 0xffffu) + (dst >> 16) + (dst & 0xffffu);
    sum = (sum & 0xffffu) + (sum >> 16);
    sum = (sum & 0xffffu) + (sum >> 16);
    uint32_t cs = ~sum & 0xffffu;
    hw[0] = 0x45u | (tos << 8) | ((L >> 8) << 16) | ((L & 0xffu) << 24);
    hw[1] = 0x00400000u;
    hw[2] = 64u | (50u << 8) | ((cs >> 8) << 16) | ((cs & 0xffu) << 24);
    hw[3] = src_img;
    hw[4] = dst_img;
}

__device__ __forceinline__ uint32_t hdr_byte(const uint32_t hw[5], uint32_t u)
{
    uint32_t w = u < 4 ? hw[0] : u < 8 ? hw[1] : u < 12 ? hw[2] : u < 16 ? hw[3] : hw[4];
    return (w >> ((u & 3u) * 8u)) & 0xffu;
}

__device__ __forceinline__ void st_v4(void *p, uint4 v)
{
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
                 "r"(v.w)
                 : "memory");
}

// Write packet bytes [d0, d0+16) (relative to the packet start) into the
// 16-B aligned destination chunk `dst`, given the record and header.
__device__ __forceinline__ void write_out_chunk(uint8_t *dst, int d0, uint32_t L, const uint4 *rec,
                                                uint32_t tos, uint32_t sa, const DevTable &T)
{
    if (d0 >= 20 && (uint32_t)d0 + 16u <= L) {
        uint32_t rb = (uint32_t)d0 - 20u;
        uint32_t sh = rb & 15u;
        uint4 lo = rec[rb >> 4];
        uint4 hi = sh ? rec[(rb >> 4) + 1] : make_uint4(0, 0, 0, 0);
        st_v4(dst, extract16(lo, hi, sh));
        return;
    }
    uint32_t hw[5];
    uint4 hd = __ldg(&T.sahdr[sa]);
    outer_header_words(tos, L, hd.z, hd.w, hw);
    const uint8_t *rb = reinterpret_cast<const uint8_t *>(rec);
#pragma unroll 1
    for (int j = 0; j < 16; j++) {
        int u = d0 + j;
        if (u < 0 || u >= (int)L) continue;
        dst[j] = (uint8_t)(u < 20 ? hdr_byte(hw, (uint32_t)u) : rb[u - 20]);
    }
}

__global__ void __launch_bounds__(1024, 1)
k_scatter(DevTable T, DevWork W, BatchArgs B)
{
    __shared__ uint32_t s_pref[TILE + 1];
    __shared__ uint32_t s_L[TILE];        // L | tos << 16
    __shared__ uint32_t s_rec[TILE];
    __shared__ uint32_t s_sa[TILE];
    __shared__ uint32_t s_scr[32];
    __shared__ uint32_t s_cnt[4];
    const uint32_t tid = threadIdx.x, lane = tid & 31u;
    const uint32_t tile = blockIdx.x;
    const uint32_t i = tile * TILE + tid;
    if (tid < 4) s_cnt[tid] = 0;

    uint32_t info = 0, L = 0, nch = 0, D = 0, sa = 0;
    uint64_t o_abs = 0;
    if (i < B.n) {
        info = W.m_info[i];
        D = B.in_len[i];
        sa = B.sa_idx[i];
        if (info & INFO_OK) {
            L = 48u + (info & 0xffffu);
            o_abs = reinterpret_cast<uint64_t>(B.out_buf) + B.out_off[i];
            nch = (uint32_t)(((o_abs + L - 1) >> 4) - (o_abs >> 4) + 1);
        }
        B.out_len[i] = (uint16_t)L;
    }
    // counters: pkts_ok, pkts_dropped, bytes_in, bytes_out (per-tile sums fit u32)
    uint32_t ok = (L != 0), dropped = (i < B.n && L == 0);
    uint32_t c0 = __reduce_add_sync(0xffffffffu, ok);
    uint32_t c1 = __reduce_add_sync(0xffffffffu, dropped);
    uint32_t c2 = __reduce_add_sync(0xffffffffu, ok ? D : 0u);
    uint32_t c3 = __reduce_add_sync(0xffffffffu, L);
    uint32_t tot;
    uint32_t my = block_exclusive_scan(nch, s_scr, &tot);   // also orders s_cnt init
    if (lane == 0) {
        atomicAdd(&s_cnt[0], c0);
        atomicAdd(&s_cnt[1], c1);
        atomicAdd(&s_cnt[2], c2);
        atomicAdd(&s_cnt[3], c3);
    }
    s_pref[tid] = my;
    if (tid == TILE - 1) s_pref[TILE] = tot;
    s_L[tid] = L | (((info >> 16) & 0xffu) << 16);
    s_rec[tid] = (info & INFO_OK) ? W.m_rec[i] : 0u;
    s_sa[tid] = sa;
    __syncthreads();
    if (tid < 4) atomicAdd(&W.counters[tid], (unsigned long long)s_cnt[tid]);
    if (tid == 4 && tile == 0) atomicAdd(&W.counters[4], 1ull);

    const uint32_t tile_first = tile * TILE;
    for (uint32_t c = tid; c < tot; c += blockDim.x) {
        uint32_t j = upper_bound_m1(s_pref, TILE, c);
        uint32_t k = c - s_pref[j];
        uint32_t Lj = s_L[j] & 0xffffu;
        uint64_t oj = reinterpret_cast<uint64_t>(B.out_buf) + B.out_off[tile_first + j];
        uint64_t A = ((oj >> 4) + k) << 4;
        int d0 = (int)((int64_t)A - (int64_t)oj);
        write_out_chunk(reinterpret_cast<uint8_t *>(A), d0, Lj, W.db + s_rec[j],
                        (s_L[j] >> 16) & 0xffu, s_sa[j], T);
    }
}

cudaError_t launch_scatter(const DevTable &T, const DevWork &W, const BatchArgs &B,
                           uint32_t n_tiles, cudaStream_t st)
{
    k_scatter<<<n_tiles, TILE, 0, st>>>(T, W, B);
    return cudaGetLastError();
}

}  // namespace nba
