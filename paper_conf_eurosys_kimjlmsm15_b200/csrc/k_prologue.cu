// k_prologue.cu -- row a1 of the hot path: per-packet validity and sizes,
// deterministic per-SA ranks (-> ESP sequence numbers), per-SA counter advance,
// and the tile-level exclusive scans that place records and AES blocks.
//
// PAPER.md:329 (§3.3): "the framework validates packet data and datablock
// fields prior to execution"; invalid packets are masked, not
// split out.  Sequence numbers: RFC 4303 §3.3.3 (per SA, +1 per packet,
// never cycling) applied in batch-index order (reading A5), so the result is
// exactly that of the sequential oracle loop.
//
// One CTA per tile of 1024 packets.  Within a warp, __match_any_sync groups
// lanes with the same SA; the per-warp groups are then merged in warp order
// through a shared histogram (deterministic: no atomics decide ranks).  The
// last CTA to finish (ticket) scans the tile histograms per SA, advances the
// SA sequence counters and scans the per-tile record / block totals.
#include "internal.cuh"

namespace nba {

__global__ void __launch_bounds__(1024, 1)
k_prologue(DevTable T, DevWork W, BatchArgs B, uint32_t n_tiles)
{
    extern __shared__ uint16_t s_hist[];             // [n_sa] counts in this tile
    __shared__ uint32_t s_scr[32];
    __shared__ uint32_t s_last;
    __shared__ uint32_t s_bin[NBINS];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t tile = blockIdx.x;
    const uint32_t i = tile * TILE + tid;
    const uint32_t n_sa = T.n_sa;

    for (uint32_t k = tid; k < n_sa; k += blockDim.x) s_hist[k] = 0;
    if (tid < NBINS) s_bin[tid] = 0;

    uint32_t s = INVALID_SA, rec16 = 0, nblk = 0;
    if (i < B.n) {
        uint32_t sa = B.sa_idx[i];
        uint32_t D = B.in_len[i];
        if (sa < n_sa && D >= MIN_D && D <= MAX_D) {
            s = sa;
            uint32_t C = esp_C(D);
            rec16 = esp_rec16(C);
            nblk = esp_nblk(C);
        }
    }
    uint32_t C_ = (s != INVALID_SA) ? esp_C(B.in_len[i]) : 0u;
    const uint32_t bin = hmac_bin(s != INVALID_SA, C_);
    const uint32_t peers = __match_any_sync(0xffffffffu, s);
    const uint32_t leader = __ffs(peers) - 1;
    const uint32_t wrank = __popc(peers & lanemask_lt());
    const uint32_t wcnt = __popc(peers);
    __syncthreads();

    // merge warp groups in warp order (deterministic ranks)
    uint32_t base = 0;
    for (uint32_t w = 0; w < blockDim.x / 32u; w++) {
        if (warp == w) {
            if (s != INVALID_SA && lane == leader) {
                base = s_hist[s];
                s_hist[s] = (uint16_t)(base + wcnt);
            }
            base = __shfl_sync(0xffffffffu, base, leader);
        }
        __syncthreads();
    }
    if (i < B.n) {
        W.lrank[i] = base + wrank;
        atomicAdd(&s_bin[bin], 1u);
    }

    for (uint32_t k = tid; k < n_sa; k += blockDim.x)
        W.hist[(size_t)tile * n_sa + k] = s_hist[k];

    uint32_t tot_rec, tot_blk;
    block_exclusive_scan(rec16, s_scr, &tot_rec);
    block_exclusive_scan(nblk, s_scr, &tot_blk);
    if (tid == 0) {
        W.tile_rec[tile] = tot_rec;
        W.tile_blk[tile] = tot_blk;
    }
    if (tid < NBINS) W.tile_bin[tile * NBINS + tid] = s_bin[tid];

    // ---- last CTA: per-SA scan over tiles, seq advance, tile scans ----------
    __threadfence();
    __syncthreads();
    if (tid == 0) s_last = (atomicAdd(&W.ctl[CTL_TICKET], 1u) == n_tiles - 1u) ? 1u : 0u;
    __syncthreads();
    if (!s_last) return;
    __threadfence();

    for (uint32_t sa = tid; sa < n_sa; sa += blockDim.x) {
        uint32_t run = 0;
        uint32_t t = 0;
        for (; t + 8 <= n_tiles; t += 8) {
            uint32_t h[8];
#pragma unroll
            for (int u = 0; u < 8; u++) h[u] = __ldcg(&W.hist[(size_t)(t + u) * n_sa + sa]);
#pragma unroll
            for (int u = 0; u < 8; u++) {
                W.hist[(size_t)(t + u) * n_sa + sa] = run;
                run += h[u];
            }
        }
        for (; t < n_tiles; t++) {
            uint32_t h = __ldcg(&W.hist[(size_t)t * n_sa + sa]);
            W.hist[(size_t)t * n_sa + sa] = run;
            run += h;
        }
        uint32_t old = T.seq[sa];
        T.seq_prev[sa] = old;
        uint32_t room = 0xffffffffu - old;
        T.seq[sa] = old + (run < room ? run : room);
    }

    uint32_t carry_rec = 0, carry_blk = 0;
    for (uint32_t t0 = 0; t0 < n_tiles; t0 += blockDim.x) {
        uint32_t t = t0 + tid;
        uint32_t vr = t < n_tiles ? __ldcg(&W.tile_rec[t]) : 0u;
        uint32_t vb = t < n_tiles ? __ldcg(&W.tile_blk[t]) : 0u;
        uint32_t sr, sb;
        uint32_t er = block_exclusive_scan(vr, s_scr, &sr);
        uint32_t eb = block_exclusive_scan(vb, s_scr, &sb);
        if (t < n_tiles) {
            W.tile_rec[t] = carry_rec + er;
            W.tile_blk[t] = carry_blk + eb;
        }
        carry_rec += sr;
        carry_blk += sb;
    }
    // HMAC length bins: bin-major, tile-minor exclusive prefix -> W.perm slots
    if (tid < NBINS) {
        uint32_t run = 0;
        for (uint32_t t = 0; t < n_tiles; t++) {
            uint32_t v = __ldcg(&W.tile_bin[t * NBINS + tid]);
            W.tile_bin[t * NBINS + tid] = run;
            run += v;
        }
        s_bin[tid] = run;
    }
    __syncthreads();
    if (tid < NBINS) {
        uint32_t off = 0;
        for (uint32_t b = 0; b < tid; b++) off += s_bin[b];
        for (uint32_t t = 0; t < n_tiles; t++) W.tile_bin[t * NBINS + tid] += off;
    }
    if (tid == 0) {
        W.ctl[CTL_TOTAL_REC] = carry_rec;
        W.ctl[CTL_TOTAL_BLK] = carry_blk;
        W.ctl[CTL_TICKET] = 0;            // re-arm for the next batch (stream-ordered)
    }
}

cudaError_t launch_prologue(const DevTable &T, const DevWork &W, const BatchArgs &B,
                            uint32_t n_tiles, cudaStream_t st)
{
    size_t smem = ((size_t)T.n_sa * 2 + 15) & ~(size_t)15;
    k_prologue<<<n_tiles, TILE, smem, st>>>(T, W, B, n_tiles);
    return cudaGetLastError();
}

cudaError_t setup_prologue_attributes(uint32_t n_sa)
{
    size_t smem = ((size_t)n_sa * 2 + 15) & ~(size_t)15;
    if (smem > 48 * 1024)
        return cudaFuncSetAttribute(k_prologue, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)smem);
    return cudaSuccess;
}

}  // namespace nba
