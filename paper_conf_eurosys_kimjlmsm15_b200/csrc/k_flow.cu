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
// One thread per packet (flow_lookup_one, fused_common.cuh; the fused kernel
// runs the same function in its prologue when the caller passes no sa_idx).
#include "fused_common.cuh"

namespace nba {

__global__ void __launch_bounds__(256)
k_flow_lookup(const uint4 *__restrict__ table, uint32_t mask, FlowArgs A)
{
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= A.n) return;
    A.sa_idx[i] = flow_lookup_one(table, mask, A.in_buf + A.in_off[i], A.in_len[i]);
}

cudaError_t launch_flow_lookup(const uint4 *table, uint32_t mask, const FlowArgs &A, cudaStream_t st)
{
    k_flow_lookup<<<(A.n + 255u) / 256u, 256, 0, st>>>(table, mask, A);
    return cudaGetLastError();
}

}  // namespace nba
