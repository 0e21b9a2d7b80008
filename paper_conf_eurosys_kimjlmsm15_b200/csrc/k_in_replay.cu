// k_in_replay.cu -- ESP inbound, steps 2 and 3: the RFC 4303
// §3.4.3 anti-replay decision for a whole batch at once, bit-exact with the
// sequential receiver (oracle_process_inbound), and the per-SA window update.
//
// Sequential rule (window W = 64, right edge `top`, bit d <-> number top - d):
// packet j of SA s passes iff q != 0 and (q > top, or top - q < W and q not yet
// marked); the window is updated only for packets that pass AND authenticate.
// Parallel form used here: let A = the packets with a
// valid format and ICV.  Packets outside A never move the window, and a packet
// of A that fails the check has q <= top, so the edge seen by packet j is
//     top_j = max(top_0, max{ q_k : k < j, k in A, same SA })     (a prefix max)
// and j passes iff q != 0 and (q > top_j, or top_j - q < W, q is not marked in
// the window at batch start, and no k < j in A of the same SA has q_k = q).
// (If such a k exists and passed, j is a duplicate; if it failed, it was too old
// or itself a duplicate, and so is j.)  The first-index test uses a hash of
// (s, q) -> min k over A.  The final window: top' = max(top_0, max over A) and
// the start bitmap shifted by top' - top_0, OR the bits of the accepted numbers.
//
// k_in_replay: one CTA per tile of PTILE packets: warp-segmented prefix max by
// SA (__match_any_sync), then each group looks up its SA among the other warps'
// groups (earlier warps raise its prefix); per-tile per-SA max into an SA-major
// matrix; hash inserts.  Then (grid barrier when the grid is
// co-resident, else the last CTA) one warp per SA scans its row (exclusive
// prefix max) and moves the window edge.
// k_in_decide: one thread per packet: status, out_len, window bits, counters.
#include "in_replay.cuh"

namespace nba {

__device__ __forceinline__ void in_grid_barrier(uint32_t *count, uint32_t *gen)
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

__global__ void __launch_bounds__(PTILE)
k_in_replay(DevTable T, InState S, InBatchArgs B, uint32_t n_tiles, uint32_t hmask, bool gridsync)
{
    constexpr uint32_t NW = PTILE / 32u;
    constexpr uint32_t HS = 2u * PTILE;                  // tile hash: <= PTILE distinct SAs
    __shared__ uint32_t s_hkey[HS];                       // SA in the slot (INVALID_SA = free)
    __shared__ uint32_t s_hmax[HS][NW];                   // the SA's group max in warp w
    __shared__ uint32_t s_hmask[HS];                      // warps that hold a group of the SA
    __shared__ uint32_t s_last;
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t tile = blockIdx.x;
    const uint32_t i = tile * PTILE + tid;
    const uint32_t n_sa = T.n_sa;
    for (uint32_t k = tid; k < HS; k += PTILE) {
        s_hkey[k] = INVALID_SA;
        s_hmask[k] = 0;
    }
    // k_in_fused's flags / sequence numbers are complete after this
    asm volatile("griddepcontrol.wait;" ::: "memory");

    // group by SA every packet that reaches the replay check (valid format);
    // only members of A (authenticated) contribute their number, the rest 0
    uint32_t key = INVALID_SA, q = 0;
    bool inA = false;
    if (i < B.n) {
        const uint32_t f = S.flags[i];
        if (f & INF_FMT) {
            key = B.sa_idx[i];
            inA = (f & INF_ICV) != 0;
            q = inA ? S.seq[i] : 0u;
        }
    }
    const uint32_t peers = __match_any_sync(0xffffffffu, key);
    const uint32_t lt = peers & lanemask_lt();
    const uint32_t mex = group_prefix_max(lt, q);   // max over earlier lanes of the group
    const uint32_t leader = __ffs(peers) - 1;
    const uint32_t hi_lane = 31u - __clz(peers);
    const uint32_t gmax = __shfl_sync(0xffffffffu, max(mex, q), hi_lane);
    __syncthreads();   // tile hash initialised

    // merge the warps' groups of the same SA through a small shared hash:
    // the group leader claims the SA's slot and records its warp's group max;
    // earlier warps then raise the prefix, and the last warp holding the SA
    // writes the tile maximum (any number of SAs per table)
    uint32_t slot = 0;
    if (key != INVALID_SA && lane == leader) {
        slot = (key * 0x9E3779B1u) >> 23;               // 9 bits -> HS = 512 slots
        while (true) {
            const uint32_t old = atomicCAS(&s_hkey[slot], INVALID_SA, key);
            if (old == INVALID_SA || old == key) break;
            slot = (slot + 1u) & (HS - 1u);
        }
        s_hmax[slot][warp] = gmax;
        atomicOr(&s_hmask[slot], 1u << warp);
    }
    slot = __shfl_sync(0xffffffffu, slot, leader);
    __syncthreads();
    uint32_t base = 0;
    bool later = false;
    if (key != INVALID_SA) {
        const uint32_t m = s_hmask[slot];
#pragma unroll
        for (uint32_t w = 0; w < NW; w++)
            if (w < warp && ((m >> w) & 1u)) base = max(base, s_hmax[slot][w]);
        later = (m >> (warp + 1u)) != 0u;
    }
    if (i < B.n) S.lmax[i] = max(base, mex);
    if (key != INVALID_SA) {
        // per-tile SA maxima, nonzero only (0 is the identity: top_0 >= 0)
        const uint32_t tmax = max(base, gmax);
        if (!later && lane == hi_lane && tmax != 0u) S.hmax[(size_t)key * n_tiles + tile] = tmax;
    }
    if (inA) replay_hash_insert(S, key, q, i, hmask);   // (s, q) -> smallest index in A

    if (gridsync) {
        in_grid_barrier(&S.ctl[1], &S.ctl[2]);
        asm volatile("griddepcontrol.launch_dependents;");
        scan_all_rows(S, n_sa, warp * gridDim.x + tile, gridDim.x * (PTILE / 32u), n_tiles, lane);
    } else {
        __threadfence();
        __syncthreads();
        if (tid == 0) s_last = (atomicAdd(&S.ctl[0], 1u) == n_tiles - 1u) ? 1u : 0u;
        __syncthreads();
        asm volatile("griddepcontrol.launch_dependents;");
        if (!s_last) return;
        __threadfence();
        scan_all_rows(S, n_sa, warp, PTILE / 32u, n_tiles, lane);
        __syncthreads();
        if (tid == 0) S.ctl[0] = 0;
    }
}

constexpr uint32_t DEC_THREADS = 256;

__global__ void __launch_bounds__(DEC_THREADS)
k_in_decide(DevTable T, InState S, InBatchArgs B, uint32_t n_tiles, uint32_t hmask)
{
    __shared__ unsigned long long s_cnt[N_IN_COUNTERS - 1];
    const uint32_t tid = threadIdx.x, lane = tid & 31u;
    const uint32_t i = blockIdx.x * DEC_THREADS + tid;
    if (tid < N_IN_COUNTERS - 1) s_cnt[tid] = 0;
    asm volatile("griddepcontrol.wait;" ::: "memory");
    __syncthreads();

    uint32_t st = 0xffu, D = 0, Lin = 0;
    if (i < B.n) {
        const uint32_t s = B.sa_idx[i];
        const uint32_t f = S.flags[i];
        if (s >= T.n_sa) {
            st = ST_DROP_SA;
        } else if (!(f & INF_FMT)) {
            st = ST_DROP_FORMAT;
        } else {
            const uint32_t q = S.seq[i];
            const uint32_t t0 = S.top_prev[s];
            const unsigned long long b0 = S.bmp_prev[s];
            const uint32_t tj = max(t0, max(S.pmx[(size_t)s * n_tiles + i / PTILE], S.lmax[i]));
            st = replay_decide(S, s, i, f, q, t0, b0, tj, S.top[s], hmask);
            if (st == ST_OK) {
                D = f & 0xffffu;
                Lin = B.in_len[i];
            }
        }
        B.out_len[i] = (uint16_t)D;
        if (B.status) B.status[i] = (uint8_t)st;
    }
    // counters: pkts_ok, drop_sa, drop_format, drop_replay, drop_auth, drop_trailer,
    // bytes_in, bytes_out (+ batches by block 0)
#pragma unroll
    for (uint32_t k = 0; k < 6; k++) {
        const uint32_t c = __reduce_add_sync(0xffffffffu, st == k ? 1u : 0u);
        if (lane == 0 && c) atomicAdd(&s_cnt[k], (unsigned long long)c);
    }
    const uint32_t bi = __reduce_add_sync(0xffffffffu, Lin);
    const uint32_t bo = __reduce_add_sync(0xffffffffu, D);
    if (lane == 0 && bi) atomicAdd(&s_cnt[6], (unsigned long long)bi);
    if (lane == 0 && bo) atomicAdd(&s_cnt[7], (unsigned long long)bo);
    __syncthreads();
    if (tid < N_IN_COUNTERS - 1 && s_cnt[tid]) atomicAdd(&S.counters[tid], s_cnt[tid]);
    if (tid == 0 && blockIdx.x == 0) atomicAdd(&S.counters[N_IN_COUNTERS - 1], 1ull);
}

static cudaError_t launch_pdl(const void *fn, dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                              void **args)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelExC(&cfg, fn, args);
}

cudaError_t launch_in_replay(const DevTable &T, const InState &S, const InBatchArgs &B,
                             uint32_t n_tiles, uint32_t hmask, bool gridsync, cudaStream_t st)
{
    DevTable t = T;
    InState s = S;
    InBatchArgs b = B;
    void *args[] = {&t, &s, &b, &n_tiles, &hmask, &gridsync};
    return launch_pdl((const void *)k_in_replay, dim3(n_tiles), dim3(PTILE), 0, st, args);
}

cudaError_t launch_in_decide(const DevTable &T, const InState &S, const InBatchArgs &B,
                             uint32_t n_tiles, uint32_t hmask, cudaStream_t st)
{
    DevTable t = T;
    InState s = S;
    InBatchArgs b = B;
    void *args[] = {&t, &s, &b, &n_tiles, &hmask};
    return launch_pdl((const void *)k_in_decide, dim3((B.n + DEC_THREADS - 1) / DEC_THREADS),
                      dim3(DEC_THREADS), 0, st, args);
}

cudaError_t setup_in_fused_attributes();

cudaError_t setup_inbound_attributes(uint32_t n_sa, uint32_t max_tiles, int num_sms, bool *gridsync)
{
    cudaError_t e = setup_in_fused_attributes();
    if (e != cudaSuccess) return e;
    (void)n_sa;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_in_replay, PTILE, 0);
    if (e != cudaSuccess) return e;
    *gridsync = (uint64_t)per_sm * (uint64_t)num_sms >= (uint64_t)max_tiles;
    return cudaSuccess;
}

}  // namespace nba
