// k_prologue.cu -- row a1 of the hot path: per-packet validity and sizes,
// deterministic per-SA ranks (-> ESP sequence numbers), the per-SA counter
// advance, and (unfused pipeline only) the tile-level scans that place records
// and AES blocks in the datablock.
//
// PAPER.md:329 (§3.3): "the framework validates packet data and datablock
// fields prior to execution"; invalid packets are masked, not
// split out.  Sequence numbers: RFC 4303 §3.3.3 (per SA, +1 per packet,
// never cycling) applied in batch-index order (reading A5), so the result is
// exactly that of the sequential oracle loop.
//
// Phase 1, one CTA per tile of PTILE = 256 packets: __match_any_sync groups
// the lanes of a warp by SA; the 8 warps' groups are merged in warp order
// through a shared histogram (deterministic: no atomic decides a rank).  The
// tile writes its per-SA counts (u16) and each packet's within-tile rank.
// Phase 2, after a grid-wide barrier (all tiles are co-resident: 256-thread
// CTAs with a 2 KB histogram): one warp per SA scans that SA's column of tile
// counts with shuffles (-> per-tile exclusive prefixes) and advances the SA's
// sequence counter.  If the grid could not be co-resident (very many SAs),
// the last CTA to finish does phase 2 alone instead.
#include "internal.cuh"

namespace nba {

static size_t prologue_smem(uint32_t n_sa) { return ((size_t)n_sa * 2 + 15) & ~(size_t)15; }

// Sense-reversing grid barrier over gridDim.x co-resident CTAs.
__device__ __forceinline__ void grid_barrier(uint32_t *count, uint32_t *gen)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        const uint32_t g = *reinterpret_cast<volatile uint32_t *>(gen);
        __threadfence();
        if (atomicAdd(count, 1u) == gridDim.x - 1u) {
            *reinterpret_cast<volatile uint32_t *>(count) = 0;
            __threadfence();
            atomicAdd(gen, 1u);
        } else {
            while (*reinterpret_cast<volatile uint32_t *>(gen) == g) __nanosleep(32);
        }
        __threadfence();
    }
    __syncthreads();
}

// Unfused pipeline only: exclusive scans of the per-tile record / AES-block
// totals and of the HMAC length bins (bin-major, tile-minor).
__device__ __forceinline__ void scan_tile_totals(const DevWork &W, uint32_t n_tiles, uint32_t *s_scr)
{
    const uint32_t tid = threadIdx.x;
    uint32_t carry_rec = 0, carry_blk = 0;
    for (uint32_t t0 = 0; t0 < n_tiles; t0 += blockDim.x) {
        const uint32_t t = t0 + tid;
        const uint32_t vr = t < n_tiles ? __ldcg(&W.tile_rec[t]) : 0u;
        const uint32_t vb = t < n_tiles ? __ldcg(&W.tile_blk[t]) : 0u;
        uint32_t sr, sb;
        const uint32_t er = block_exclusive_scan(vr, s_scr, &sr);
        const uint32_t eb = block_exclusive_scan(vb, s_scr, &sb);
        if (t < n_tiles) {
            W.tile_rec[t] = carry_rec + er;
            W.tile_blk[t] = carry_blk + eb;
        }
        carry_rec += sr;
        carry_blk += sb;
    }
    const uint32_t tot = n_tiles * NBINS;
    uint32_t carry = 0;
    for (uint32_t e0 = 0; e0 < tot; e0 += blockDim.x) {
        const uint32_t e = e0 + tid;
        const uint32_t b = e / n_tiles, t = e % n_tiles;
        const uint32_t v = e < tot ? __ldcg(&W.tile_bin[t * NBINS + b]) : 0u;
        uint32_t s;
        const uint32_t ex = block_exclusive_scan(v, s_scr, &s);
        if (e < tot) W.tile_bin[t * NBINS + b] = carry + ex;
        carry += s;
    }
    if (tid == 0) {
        W.ctl[CTL_TOTAL_REC] = carry_rec;
        W.ctl[CTL_TOTAL_BLK] = carry_blk;
    }
}

__global__ void __launch_bounds__(PTILE)
k_prologue(DevTable T, DevWork W, BatchArgs B, uint32_t n_tiles, bool unfused, bool gridsync)
{
    extern __shared__ uint16_t s_hist[];             // [n_sa] counts in this tile
    __shared__ uint32_t s_scr[32];
    __shared__ uint32_t s_last;
    __shared__ uint32_t s_bin[NBINS];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t tile = blockIdx.x;
    const uint32_t i = tile * PTILE + tid;
    const uint32_t n_sa = T.n_sa;
    unsigned long long *tr = W.trace ? W.trace + (size_t)W.trace_pro : nullptr;
    if (tr && tid == 0) atomicMin(&tr[0], gtimer());

    for (uint32_t k = tid; k < n_sa; k += PTILE) s_hist[k] = 0;
    if (tid < NBINS) s_bin[tid] = 0;

    uint32_t s = INVALID_SA, rec16 = 0, nblk = 0, C = 0;
    if (i < B.n) {
        const uint32_t sa = B.sa_idx[i];
        const uint32_t D = B.in_len[i];
        if (sa < n_sa && D >= MIN_D && D <= MAX_D) {
            s = sa;
            C = esp_C(D);
            rec16 = esp_rec16(C);
            nblk = esp_nblk(C);
        }
    }
    const uint32_t peers = __match_any_sync(0xffffffffu, s);
    const uint32_t leader = __ffs(peers) - 1;
    const uint32_t wrank = __popc(peers & lanemask_lt());
    const uint32_t wcnt = __popc(peers);
    __syncthreads();

    // merge the warps' groups in warp order (deterministic ranks)
    uint32_t base = 0;
#pragma unroll 1
    for (uint32_t w = 0; w < PTILE / 32u; w++) {
        if (warp == w) {
            if (s != INVALID_SA && lane == leader) {
                base = s_hist[s];
                s_hist[s] = (uint16_t)(base + wcnt);
            }
            base = __shfl_sync(0xffffffffu, base, leader);
        }
        __syncthreads();
    }
    if (i < B.n) W.lrank[i] = base + wrank;
    // SA-major tile counts, nonzero entries only (the column scan re-zeroes what
    // it reads, so the matrix is all-zero between batches): the packet with the
    // tile's highest rank for its SA writes that SA's count
    if (s != INVALID_SA && base + wrank + 1u == s_hist[s])
        W.hist16[(size_t)s * n_tiles + tile] = s_hist[s];

    if (unfused) {
        if (i < B.n) atomicAdd(&s_bin[hmac_bin(s != INVALID_SA, C)], 1u);
        uint32_t tot_rec, tot_blk;
        block_exclusive_scan(rec16, s_scr, &tot_rec);
        block_exclusive_scan(nblk, s_scr, &tot_blk);
        if (tid == 0) {
            W.tile_rec[tile] = tot_rec;
            W.tile_blk[tile] = tot_blk;
        }
        if (tid < NBINS) W.tile_bin[tile * NBINS + tid] = s_bin[tid];
    }
    if (tr && tid == 0) atomicMax(&tr[1], gtimer());

    if (gridsync) {
        // ---- phase 2 on every CTA: one warp per SA column -------------------
        grid_barrier(&W.ctl[CTL_BAR_COUNT], &W.ctl[CTL_BAR_GEN]);
        if (tr && tid == 0 && tile == 0) tr[2] = gtimer();
        // let the dependent (fused) kernel launch and stage its tables; it waits
        // for this grid's completion before reading our outputs
        asm volatile("griddepcontrol.launch_dependents;");
        scan_all_columns(T, W, tile * (PTILE / 32u) + warp, gridDim.x * (PTILE / 32u), n_tiles, lane);
        if (unfused && tile == 0) scan_tile_totals(W, n_tiles, s_scr);
    } else {
        // ---- phase 2 on the last CTA to finish phase 1 -----------------------
        __threadfence();
        __syncthreads();
        if (tid == 0) s_last = (atomicAdd(&W.ctl[CTL_TICKET], 1u) == n_tiles - 1u) ? 1u : 0u;
        __syncthreads();
        asm volatile("griddepcontrol.launch_dependents;");
        if (!s_last) return;
        __threadfence();
        if (tr && tid == 0) tr[2] = gtimer();
        scan_all_columns(T, W, warp, PTILE / 32u, n_tiles, lane);
        if (unfused) scan_tile_totals(W, n_tiles, s_scr);
        __syncthreads();
        if (tid == 0) W.ctl[CTL_TICKET] = 0;            // re-arm for the next batch
    }
    if (tr) {
        __syncthreads();
        if (tid == 0) atomicMax(&tr[3], gtimer());
    }
}

cudaError_t launch_prologue(const DevTable &T, const DevWork &W, const BatchArgs &B,
                            uint32_t n_tiles, bool unfused, bool gridsync, cudaStream_t st)
{
    k_prologue<<<n_tiles, PTILE, prologue_smem(T.n_sa), st>>>(T, W, B, n_tiles, unfused, gridsync);
    return cudaGetLastError();
}

cudaError_t setup_prologue_attributes(uint32_t n_sa, uint32_t max_tiles, int num_sms, bool *gridsync)
{
    const size_t smem = prologue_smem(n_sa);
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(k_prologue, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)smem);
        if (e != cudaSuccess) return e;
    }
    int per_sm = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_prologue, PTILE, smem);
    if (e != cudaSuccess) return e;
    // grid-wide barrier only if every tile of the largest batch is co-resident
    *gridsync = (uint64_t)per_sm * (uint64_t)num_sms >= (uint64_t)max_tiles;
    return cudaSuccess;
}

}  // namespace nba
