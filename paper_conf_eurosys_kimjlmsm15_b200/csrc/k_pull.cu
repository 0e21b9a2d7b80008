// k_pull.cu -- the host path's metadata pull (nba_ipsec_process_batch_host with
// NBA_IPSEC_HOST_META=pull; measured slower than reading in place, kept as the A/B):
// the per-packet arrays in_off, sa_idx, out_off (u32) and in_len (u16), in
// page-locked host memory the device addresses, read over PCIe by every
// thread of a grid-stride loop (4-byte words, a warp's 32 loads one 128-byte
// request) into the staging slot on the device.  One launch instead of four
// copy-engine copies (whose per-copy cost is most of their time at 65,536
// packets, tools/pcie_probe.py), and the main kernels then read device memory.
#include <algorithm>

#include "internal.cuh"

namespace nba {

__global__ void __launch_bounds__(256)
k_pull_meta(const uint32_t *__restrict__ h_in_off, const uint32_t *__restrict__ h_sa,
            const uint32_t *__restrict__ h_out_off, const uint16_t *__restrict__ h_in_len,
            uint32_t *__restrict__ in_off, uint32_t *__restrict__ sa, uint32_t *__restrict__ out_off,
            uint16_t *__restrict__ in_len, uint32_t n)
{
    const uint32_t stride = gridDim.x * blockDim.x;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const uint32_t a = h_in_off[i], b = h_sa[i], c = h_out_off[i];
        const uint16_t d = h_in_len[i];
        in_off[i] = a;
        sa[i] = b;
        out_off[i] = c;
        in_len[i] = d;
    }
}

cudaError_t launch_pull_meta(const uint32_t *h_in_off, const uint32_t *h_sa, const uint32_t *h_out_off,
                             const uint16_t *h_in_len, uint32_t *in_off, uint32_t *sa, uint32_t *out_off,
                             uint16_t *in_len, uint32_t n, int num_sms, cudaStream_t st)
{
    if (n == 0) return cudaSuccess;
    const uint32_t blocks = std::min<uint32_t>((n + 255u) / 256u, (uint32_t)num_sms * 8u);
    k_pull_meta<<<blocks, 256, 0, st>>>(h_in_off, h_sa, h_out_off, h_in_len, in_off, sa, out_off, in_len, n);
    return cudaGetLastError();
}

}  // namespace nba
