// k_aes.cu -- row a3 of the hot path (unfused pipeline): AES-128-CTR over the
// ESP payload of every record, in place, one thread per 16-byte block.
//
// PAPER.md:389 (§4.1): "IPsec encryption uses ... AES-128CTR to encrypt"; the
// counter block is nonce || IV || BE32(k+1) (RFC 3686 §4, reading A7) with
// IV = BE64(seq) (A6).  PAPER.md:737: on the GTX 680 this kernel took
// ~40 us of the ~140 us of kernel time per offload.
//
// Persistent grid (one 512-thread CTA per SM, 128 KB of replicated T-tables
// built once per CTA).  CTA c owns AES blocks [c*per, (c+1)*per); its first
// packet was located by k_gather (W.aes_start).  Blocks are mapped to packets
// through a window of 512 packet start offsets staged in shared memory.
#include "aes_round.cuh"

namespace nba {

constexpr int AES_THREADS = 512;

__global__ void __launch_bounds__(AES_THREADS, 1)
k_aes(DevTable T, DevWork W, BatchArgs B)
{
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ uint32_t s_start[AES_THREADS + 1];
    __shared__ uint32_t s_next;
    const uint32_t tid = threadIdx.x;
    const uint32_t lane4 = (tid & 31u) * 4u;

    aes_tables_to_smem(smem, T.te0);

    const uint32_t total = W.ctl[CTL_TOTAL_BLK];
    const uint32_t per = (total + gridDim.x - 1) / gridDim.x;
    uint32_t g = blockIdx.x * per;
    const uint32_t gend = min(g + per, total);
    uint32_t p = (g < gend) ? W.aes_start[blockIdx.x] : 0u;
    __syncthreads();

    while (g < gend) {
        uint32_t pk = p + tid;
        s_start[tid] = pk < B.n ? W.m_blk[pk] : total;
        if (tid == 0) s_start[AES_THREADS] = (p + AES_THREADS < B.n) ? W.m_blk[p + AES_THREADS] : total;
        __syncthreads();
        uint32_t wend = min(g + (uint32_t)AES_THREADS, gend);
        wend = min(wend, s_start[AES_THREADS]);
        uint32_t my = g + tid;
        if (my < wend) {
            uint32_t k = upper_bound_m1(s_start, AES_THREADS, my);
            uint32_t pkt = p + k;
            uint32_t bi = my - s_start[k];
            uint32_t info = W.m_info[pkt];
            if (info & INFO_OK) {
                uint32_t sa = B.sa_idx[pkt];
                uint32_t q = W.m_seq[pkt];
                uint4 *dst = W.db + (size_t)W.m_rec[pkt] + 1u + bi;
                uint4 rk[11];
#pragma unroll
                for (int r = 0; r < 11; r++) rk[r] = __ldg(&T.rk[(size_t)sa * 11u + r]);
                uint32_t nonce = __ldg(&T.sahdr[sa].y);
                uint4 ks = aes128_encrypt_block(smem, lane4, rk, nonce, 0u, bswap32(q),
                                                bswap32(bi + 1u));
                uint4 d = *dst;
                d.x ^= ks.x;
                d.y ^= ks.y;
                d.z ^= ks.z;
                d.w ^= ks.w;
                *dst = d;
            }
        }
        if (tid == 0) s_next = p + upper_bound_m1(s_start, AES_THREADS + 1, wend);
        __syncthreads();
        p = s_next;
        g = wend;
    }
}

int aes_grid(int num_sms) { return num_sms; }

cudaError_t launch_aes(const DevTable &T, const DevWork &W, const BatchArgs &B, int grid,
                       cudaStream_t st)
{
    k_aes<<<grid, AES_THREADS, AES_TABLE_BYTES, st>>>(T, W, B);
    return cudaGetLastError();
}

cudaError_t setup_aes_attributes()
{
    return cudaFuncSetAttribute(k_aes, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)AES_TABLE_BYTES);
}

}  // namespace nba
