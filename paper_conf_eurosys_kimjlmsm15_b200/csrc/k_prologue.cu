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

// Dynamic shared memory of the prologue: the tile histogram (u16 per SA), or
// -- when it fits -- the whole [tiles x SAs] u16 histogram for the last CTA's
// column scan.
static size_t prologue_smem(uint32_t n_sa, uint32_t n_tiles)
{
    size_t tile = ((size_t)n_sa * 2 + 15) & ~(size_t)15;
    size_t all = ((size_t)n_sa * n_tiles * 2 + 15) & ~(size_t)15;
    const size_t cap = 200u * 1024u;
    return all <= cap ? (all > tile ? all : tile) : tile;
}

__global__ void __launch_bounds__(1024, 1)
k_prologue(DevTable T, DevWork W, BatchArgs B, uint32_t n_tiles, bool unfused, uint32_t smem_bytes)
{
    extern __shared__ uint16_t s_hist[];             // [n_sa] counts in this tile
    __shared__ uint32_t s_scr[32];
    __shared__ uint32_t s_last;
    __shared__ uint32_t s_bin[NBINS];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t tile = blockIdx.x;
    const uint32_t i = tile * TILE + tid;
    const uint32_t n_sa = T.n_sa;

    unsigned long long *tr = W.trace ? W.trace + (size_t)W.trace_pro : nullptr;
    if (tr && tid == 0) atomicMin(&tr[0], gtimer());
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
        W.hist16[(size_t)tile * n_sa + k] = s_hist[k];
    // let the dependent (fused) kernel launch and build its tables meanwhile;
    // it waits for this grid's completion before reading our outputs
    asm volatile("griddepcontrol.launch_dependents;");

    uint32_t tot_rec, tot_blk;
    block_exclusive_scan(rec16, s_scr, &tot_rec);
    block_exclusive_scan(nblk, s_scr, &tot_blk);
    if (unfused) {
        if (tid == 0) {
            W.tile_rec[tile] = tot_rec;
            W.tile_blk[tile] = tot_blk;
        }
        if (tid < NBINS) W.tile_bin[tile * NBINS + tid] = s_bin[tid];
    }

    // ---- last CTA: per-SA scan over tiles, seq advance, tile scans ----------
    __threadfence();
    __syncthreads();
    if (tr && tid == 0) atomicMax(&tr[1], gtimer());
    if (tid == 0) s_last = (atomicAdd(&W.ctl[CTL_TICKET], 1u) == n_tiles - 1u) ? 1u : 0u;
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    if (tr && tid == 0) tr[2] = gtimer();

    // per-SA exclusive scan down the tile columns -> hpfx, and the SA counter advance
    const size_t cells = (size_t)n_tiles * n_sa;
    if (cells * 2 <= smem_bytes) {
        // whole histogram into shared memory with 16-byte loads, then scan there
        uint16_t *m = s_hist;
        const size_t n16 = cells / 8;                  // cells is a multiple of 8 (n_sa even)
        const uint4 *src = reinterpret_cast<const uint4 *>(W.hist16);
        for (size_t e0 = 0; e0 < n16; e0 += 4u * blockDim.x) {
            uint4 v[4];
#pragma unroll
            for (int u = 0; u < 4; u++) {
                size_t e = e0 + tid + (size_t)u * blockDim.x;
                v[u] = e < n16 ? __ldcg(&src[e]) : make_uint4(0, 0, 0, 0);
            }
#pragma unroll
            for (int u = 0; u < 4; u++) {
                size_t e = e0 + tid + (size_t)u * blockDim.x;
                if (e < n16) reinterpret_cast<uint4 *>(m)[e] = v[u];
            }
        }
        for (size_t e = n16 * 8 + tid; e < cells; e += blockDim.x) m[e] = __ldcg(&W.hist16[e]);
        __syncthreads();
        for (uint32_t sa = tid; sa < n_sa; sa += blockDim.x) {
            uint32_t run = 0;
            for (uint32_t t = 0; t < n_tiles; t++) {
                const uint32_t h = m[(size_t)t * n_sa + sa];
                W.hpfx[(size_t)t * n_sa + sa] = run;
                run += h;
            }
            const uint32_t old = T.seq[sa];
            T.seq_prev[sa] = old;
            const uint32_t room = 0xffffffffu - old;
            T.seq[sa] = old + (run < room ? run : room);
        }
    } else {
        for (uint32_t sa = tid; sa < n_sa; sa += blockDim.x) {
            uint32_t run = 0;
            for (uint32_t t0 = 0; t0 < n_tiles; t0 += 16) {
                uint32_t h[16];
#pragma unroll
                for (int u = 0; u < 16; u++)
                    h[u] = (t0 + u < n_tiles) ? __ldcg(&W.hist16[(size_t)(t0 + u) * n_sa + sa]) : 0u;
#pragma unroll
                for (int u = 0; u < 16; u++) {
                    if (t0 + u < n_tiles) W.hpfx[(size_t)(t0 + u) * n_sa + sa] = run;
                    run += h[u];
                }
            }
            const uint32_t old = T.seq[sa];
            T.seq_prev[sa] = old;
            const uint32_t room = 0xffffffffu - old;
            T.seq[sa] = old + (run < room ? run : room);
        }
    }
    __syncthreads();

    uint32_t carry_rec = 0, carry_blk = 0;
    if (unfused) {
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
        // HMAC length bins, bin-major / tile-minor order: one flattened block scan
        const uint32_t tot = n_tiles * NBINS;
        uint32_t carry = 0;
        for (uint32_t e0 = 0; e0 < tot; e0 += blockDim.x) {
            uint32_t e = e0 + tid;
            uint32_t b = e / n_tiles, t = e % n_tiles;
            uint32_t v = e < tot ? __ldcg(&W.tile_bin[t * NBINS + b]) : 0u;
            uint32_t s;
            uint32_t ex = block_exclusive_scan(v, s_scr, &s);
            if (e < tot) W.tile_bin[t * NBINS + b] = carry + ex;
            carry += s;
        }
    }
    if (tid == 0) {
        W.ctl[CTL_TOTAL_REC] = carry_rec;
        W.ctl[CTL_TOTAL_BLK] = carry_blk;
        W.ctl[CTL_TICKET] = 0;            // re-arm for the next batch (stream-ordered)
        W.ctl[CTL_WORK] = 0;              // fused kernel's work counter
    }
    if (tr) {
        __syncthreads();
        if (tid == 0) tr[3] = gtimer();
    }
}

cudaError_t launch_prologue(const DevTable &T, const DevWork &W, const BatchArgs &B,
                            uint32_t n_tiles, bool unfused, cudaStream_t st)
{
    size_t smem = prologue_smem(T.n_sa, n_tiles);
    k_prologue<<<n_tiles, TILE, smem, st>>>(T, W, B, n_tiles, unfused, (uint32_t)smem);
    return cudaGetLastError();
}

cudaError_t setup_prologue_attributes(uint32_t n_sa, uint32_t max_tiles)
{
    size_t smem = prologue_smem(n_sa, max_tiles);
    if (smem < 200u * 1024u && (size_t)n_sa * max_tiles * 2 > smem) smem = 200u * 1024u;
    if (smem > 48 * 1024)
        return cudaFuncSetAttribute(k_prologue, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)smem);
    return cudaSuccess;
}

}  // namespace nba
