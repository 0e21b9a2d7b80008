// k_flow.cu -- flow -> SA lookup on the GPU (the step before
// the path).  PAPER.md:395 keeps one crypto context per flow, set up at
// startup; the caller registers the flows (exact inner IPv4 5-tuples) with
// nba_ipsec_set_flow_table and the packets' SA indices are found here.
//
// Per packet i (readings F1..F4): the inner datagram at
// in_buf + in_off[i] of in_len[i] bytes has a key only if it is IPv4 with
// 20 <= 4 IHL <= D; key = (src, dst, protocol, sport, dport) with the ports
// read after the IPv4 header for TCP / UDP first fragments (offset 0) when
// 4 bytes are there, else 0.  sa_idx[i] = the matching flow's SA, or
// 0xffffffff (no key / no match: the path then drops the packet).
//
// One thread per packet: one unaligned 24-byte header load (two if the header
// has options), then linear probing in the L2-resident table (16 B entries).
#include "fused_common.cuh"

namespace nba {

__global__ void __launch_bounds__(256)
k_flow_lookup(const uint4 *__restrict__ table, uint32_t mask, FlowArgs A)
{
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= A.n) return;
    uint32_t sa = INVALID_SA;
    const uint32_t D = A.in_len[i];
    if (D >= 20u) {
        const uint8_t *P = A.in_buf + A.in_off[i];
        const uintptr_t pa = reinterpret_cast<uintptr_t>(P);
        uint32_t w[6];
        load_words<6>(pa, pa + D, w);
        const uint32_t vihl = w[0] & 0xffu, ihl = vihl & 15u;
        if ((vihl >> 4) == 4u && ihl >= 5u && D >= 4u * ihl) {
            const uint32_t src = bswap32(w[3]), dst = bswap32(w[4]);
            const uint32_t proto = (w[2] >> 8) & 0xffu;
            const uint32_t frag = ((w[1] >> 8) & 0x1f00u) | (w[1] >> 24);   // bytes 6..7, 13 bits
            uint32_t ports = 0;
            if ((proto == 6u || proto == 17u) && frag == 0u && D >= 4u * ihl + 4u) {
                if (ihl == 5u) {
                    ports = bswap32(w[5]);
                } else {
                    uint32_t x[1];
                    load_words<1>(pa + 4u * ihl, pa + D, x);
                    ports = bswap32(x[0]);
                }
            }
            uint32_t h = flow_hash(src, dst, ports, proto) & mask;
            while (true) {
                const uint4 e = __ldg(&table[h]);
                if (!(e.w & FLOW_VALID)) break;
                if (e.x == src && e.y == dst && e.z == ports && (e.w & 0xffu) == proto) {
                    sa = e.w >> 16;
                    break;
                }
                h = (h + 1u) & mask;
            }
        }
    }
    A.sa_idx[i] = sa;
}

cudaError_t launch_flow_lookup(const uint4 *table, uint32_t mask, const FlowArgs &A, cudaStream_t st)
{
    k_flow_lookup<<<(A.n + 255u) / 256u, 256, 0, st>>>(table, mask, A);
    return cudaGetLastError();
}

}  // namespace nba
