// k_gather.cu -- row a2 of the hot path (unfused pipeline): finalise per-packet
// metadata (sequence number, record / block offsets) and build each ESP record
// in the datablock:
//
//   record[0,16)      BE32(spi) || BE32(seq) || IV = BE64(seq)     (RFC 4303 §2, A6)
//   record[16,16+D)   inner datagram P                             (A3)
//   record[16+D,16+C) pad 01 02 .. p, pad length p, next header 4  (RFC 4303 §2.4-2.6)
//   record[16+C,..)   zero fill (ICV goes to [16+C, 16+C+12))
//
// PAPER.md:329-343 (§3.3, Table 2): a datablock is the input byte range
// (offset, length) of each packet, staged for the accelerator; PAPER.md:737:
// on the GTX 680 the host<->device copies of this data took longer than the
// kernels -- on B200 the packets are device-resident and the "copy" is this
// coalesced on-device gather.
//
// One CTA per tile of 1024 packets; thread i of the tile finalises packet i,
// then the CTA copies the tile's records 16 bytes per thread (consecutive
// threads -> consecutive 16-B chunks -> coalesced loads and stores).
#include "internal.cuh"

namespace nba {

// T = P || pad || p || 4 ; byte b >= D of T (0 beyond C)
__device__ __forceinline__ uint32_t trailer_byte(uint32_t b, uint32_t D, uint32_t p)
{
    if (b < D + p) return b - D + 1u;
    if (b == D + p) return p;
    if (b == D + p + 1u) return 4u;
    return 0u;
}

// 16 bytes of T starting at byte `pos` for datagram `src` of D bytes.
__device__ __forceinline__ uint4 build_payload_chunk(const uint8_t *src, uint32_t D, uint32_t p,
                                                     uint32_t pos)
{
    uint4 v = make_uint4(0, 0, 0, 0);
    if (pos < D) {
        uintptr_t a = reinterpret_cast<uintptr_t>(src) + pos;
        uintptr_t base = a & ~(uintptr_t)15;
        uint32_t sh = (uint32_t)(a & 15);
        uintptr_t end = reinterpret_cast<uintptr_t>(src) + D;   // one past the last byte
        uint4 lo = ldg_nc_v4(reinterpret_cast<const void *>(base));
        uint4 hi = make_uint4(0, 0, 0, 0);
        if (sh != 0 && base + 16 < end) hi = ldg_nc_v4(reinterpret_cast<const void *>(base + 16));
        v = extract16(lo, hi, sh);
        if (pos + 16 <= D) return v;
    }
#pragma unroll
    for (uint32_t j = 0; j < 16; j++) {
        uint32_t b = pos + j;
        if (b >= D) set_byte(v, j, trailer_byte(b, D, p));
    }
    return v;
}

__global__ void __launch_bounds__(PTILE)
k_gather(DevTable T, DevWork W, BatchArgs B, uint32_t aes_grid)
{
    __shared__ uint32_t s_pref[PTILE + 1];   // record-chunk prefix within the tile
    __shared__ uint32_t s_D[PTILE];          // D | INFO_OK-bit
    __shared__ uint32_t s_sa[PTILE];
    __shared__ uint32_t s_seq[PTILE];
    __shared__ uint32_t s_scr[32];
    __shared__ uint32_t s_bin[NBINS];
    const uint32_t tid = threadIdx.x;
    const uint32_t tile = blockIdx.x;
    const uint32_t i = tile * PTILE + tid;
    const uint32_t n_sa = T.n_sa;
    if (tid < NBINS) s_bin[tid] = 0;

    uint32_t s = INVALID_SA, D = 0, C = 0, rec16 = 0, nblk = 0, info = 0, q32 = 0;
    if (i < B.n) {
        uint32_t sa = B.sa_idx[i];
        D = B.in_len[i];
        if (sa < n_sa && D >= MIN_D && D <= MAX_D) {
            s = sa;
            C = esp_C(D);
            rec16 = esp_rec16(C);
            nblk = esp_nblk(C);
            unsigned long long q = (unsigned long long)T.seq_prev[s] + 1ull +
                                   W.hpfx[(size_t)s * gridDim.x + tile] + W.lrank[i];
            q32 = (uint32_t)q;
            uint32_t tos = B.in_buf[B.in_off[i] + 1];
            info = C | (tos << 16) | (q <= 0xffffffffull ? INFO_OK : 0u);
            if (!(info & INFO_OK)) info = 0;      // sequence space exhausted -> drop
        }
    }
    uint32_t tot_rec, tot_blk;
    uint32_t my_rec = block_exclusive_scan(rec16, s_scr, &tot_rec);
    uint32_t my_blk = block_exclusive_scan(nblk, s_scr, &tot_blk);
    const uint32_t rec_base = W.tile_rec[tile];
    const uint32_t blk_base = W.tile_blk[tile];
    if (i < B.n) {
        W.m_rec[i] = rec_base + my_rec;
        W.m_blk[i] = blk_base + my_blk;
        W.m_seq[i] = q32;
        W.m_info[i] = info;
        if (i == B.n - 1) W.m_blk[B.n] = blk_base + my_blk + nblk;
        // HMAC order: counting sort by SHA-1 block count (any order is correct)
        uint32_t bin = hmac_bin(s != INVALID_SA, C);
        uint32_t r = atomicAdd(&s_bin[bin], 1u);
        W.perm[W.tile_bin[tile * NBINS + bin] + r] = i;
        // first packet of every persistent AES CTA whose range starts in this packet
        if (nblk) {
            const uint32_t total = W.ctl[CTL_TOTAL_BLK];
            const uint32_t per = (total + aes_grid - 1) / aes_grid;
            const uint32_t b0 = blk_base + my_blk;
            for (uint32_t c = (b0 + per - 1) / per; c * per < b0 + nblk && c < aes_grid; c++)
                W.aes_start[c] = i;
        }
    }
    s_pref[tid] = my_rec;
    if (tid == PTILE - 1) s_pref[PTILE] = tot_rec;
    s_D[tid] = D | (info ? INFO_OK : 0u);
    s_sa[tid] = s;
    s_seq[tid] = q32;
    __syncthreads();

    const uint32_t tile_first = tile * PTILE;
    for (uint32_t c = tid; c < tot_rec; c += blockDim.x) {
        uint32_t j = upper_bound_m1(s_pref, PTILE, c);
        uint32_t k = c - s_pref[j];
        uint32_t dd = s_D[j];
        if (!(dd & INFO_OK)) continue;            // dropped: record never read
        uint32_t Dj = dd & 0xffffu;
        uint32_t pkt = tile_first + j;
        uint4 v;
        if (k == 0) {
            uint32_t qbe = bswap32(s_seq[j]);
            v = make_uint4(__ldg(&T.sahdr[s_sa[j]].x), qbe, 0u, qbe);
        } else {
            const uint8_t *src = B.in_buf + B.in_off[pkt];
            v = build_payload_chunk(src, Dj, esp_pad(Dj), (k - 1) * 16u);
        }
        W.db[(size_t)(rec_base + s_pref[j]) + k] = v;
    }
}

cudaError_t launch_gather(const DevTable &T, const DevWork &W, const BatchArgs &B,
                          uint32_t n_tiles, uint32_t aes_grid, cudaStream_t st)
{
    k_gather<<<n_tiles, PTILE, 0, st>>>(T, W, B, aes_grid);
    return cudaGetLastError();
}

}  // namespace nba
