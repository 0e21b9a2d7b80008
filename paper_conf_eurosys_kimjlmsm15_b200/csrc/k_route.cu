// k_route.cu -- single-ingress redistribution (second half):
// when all traffic enters at one GPU, every packet must reach the GPU that owns
// its SA (SA-hash shard, owner = sa mod world, S§8(e), or the owner the
// adaptive split assigned, f4: sa_map[sa] = owner << 24 | local) before the path runs
// there.  These kernels route and pack a batch by destination so one NCCL
// all-to-all per array moves it (paper_conf_eurosys_kimjlmsm15_b200/redistribute.py):
//   k_route_tiles : per 256-packet tile, each packet's destination, its rank
//                   and byte offset among the tile's packets for that
//                   destination (warp ballots / segmented scans, warp order),
//                   and the tile's per-destination counts and bytes;
//   k_route_scan  : exclusive scans of those over tiles, and the destination
//                   regions of the send buffers (destination-major);
//   k_route_pack  : one warp per packet copies its bytes to its place and
//                   writes its length and LOCAL SA index (sa / world, or
//                   the map's low 24 bits).
// Stable: a destination receives its packets in batch-index order, so the
// per-SA sequence numbers at the owner are those of the sequential oracle.
// Packets without a valid SA (sa >= n_sa_total) are not sent (counted in slot
// `world`).
#include "internal.cuh"

namespace nba {

constexpr uint32_t RT_MAX_WORLD = 8;
constexpr uint32_t RT_TILE = 256;

struct RouteWork {
    uint32_t *dest;        // [n]   destination (world = dropped)
    uint32_t *rank;        // [n]   rank among the tile's packets of that destination
    uint32_t *brank;       // [n]   byte offset among them
    uint32_t *tcnt;        // [tiles][world+1] counts -> exclusive prefix over tiles
    unsigned long long *tbyt;   // [tiles][world+1] bytes  -> exclusive prefix over tiles
    unsigned long long *base;   // [2][world+1] region starts: packets, bytes
};

__global__ void __launch_bounds__(RT_TILE)
k_route_tiles(RouteWork R, const uint16_t *in_len, const uint32_t *sa, uint32_t n,
              uint32_t n_sa_total, const uint32_t *sa_map, uint32_t world)
{
    __shared__ uint32_t s_wc[RT_TILE / 32][RT_MAX_WORLD + 1];
    __shared__ uint32_t s_wb[RT_TILE / 32][RT_MAX_WORLD + 1];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t i = blockIdx.x * RT_TILE + tid;
    const uint32_t len = i < n ? in_len[i] : 0u;
    const uint32_t s = i < n ? sa[i] : INVALID_SA;
    // owner: s mod world (SA-hash shard) or the adaptive split's map (f4)
    uint32_t d = RT_MAX_WORLD + 1u;
    if (i < n) d = s < n_sa_total ? (sa_map ? min(__ldg(sa_map + s) >> 24, world) : s % world) : world;
    uint32_t my_rank = 0, my_brank = 0;
    for (uint32_t k = 0; k <= world; k++) {
        const uint32_t m = __ballot_sync(0xffffffffu, d == k);
        uint32_t x = d == k ? len : 0u;          // inclusive scan of lengths over the warp
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= (uint32_t)o) x += y;
        }
        if (d == k) {
            my_rank = __popc(m & lanemask_lt());
            my_brank = x - len;
        }
        if (lane == 31) {
            s_wc[warp][k] = __popc(m);
            s_wb[warp][k] = x;
        }
    }
    __syncthreads();
    if (i < n) {
        uint32_t pc = 0, pb = 0;                // earlier warps of the tile, same destination
        for (uint32_t w = 0; w < warp; w++) {
            pc += s_wc[w][d];
            pb += s_wb[w][d];
        }
        R.dest[i] = d;
        R.rank[i] = pc + my_rank;
        R.brank[i] = pb + my_brank;
    }
    if (tid <= world) {
        uint32_t c = 0, b = 0;
        for (uint32_t w = 0; w < RT_TILE / 32; w++) {
            c += s_wc[w][tid];
            b += s_wb[w][tid];
        }
        R.tcnt[blockIdx.x * (world + 1u) + tid] = c;
        R.tbyt[blockIdx.x * (world + 1u) + tid] = b;
    }
}

// One CTA: exclusive scans over tiles per destination, then region bases.
__global__ void __launch_bounds__(32 * (RT_MAX_WORLD + 1))
k_route_scan(RouteWork R, uint32_t n_tiles, uint32_t world, unsigned long long *dest_counts,
             unsigned long long *dest_bytes, const nba_ipsec_peer_rx *rx)
{
    __shared__ unsigned long long s_tc[RT_MAX_WORLD + 1], s_tb[RT_MAX_WORLD + 1];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    // warp k scans destination k's column (world + 1 <= 9 columns, 8 warps:
    // warp 0 also takes column 8)
    constexpr uint32_t U = 8;                  // 8 x 32 tiles per pass, loads issued together
    for (uint32_t k = warp; k <= world; k += blockDim.x >> 5) {   // one warp per column
        unsigned long long cc = 0, cb = 0;
        for (uint32_t t0 = 0; t0 < n_tiles; t0 += 32u * U) {
            uint32_t cu[U];
            unsigned long long bu[U];
#pragma unroll
            for (uint32_t u = 0; u < U; u++) {
                const uint32_t t = t0 + 32u * u + lane;
                cu[u] = t < n_tiles ? R.tcnt[t * (world + 1u) + k] : 0u;
                bu[u] = t < n_tiles ? R.tbyt[t * (world + 1u) + k] : 0ull;
            }
            // the U inclusive scans are independent (their shuffle chains
            // interleave); the carries are applied afterwards
            uint32_t xc[U];
            unsigned long long xb[U];
#pragma unroll
            for (uint32_t u = 0; u < U; u++) {
                xc[u] = cu[u];
                xb[u] = bu[u];
            }
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
                for (uint32_t u = 0; u < U; u++) {
                    const uint32_t yc = __shfl_up_sync(0xffffffffu, xc[u], o);
                    const unsigned long long yb = __shfl_up_sync(0xffffffffu, xb[u], o);
                    if (lane >= (uint32_t)o) {
                        xc[u] += yc;
                        xb[u] += yb;
                    }
                }
            }
#pragma unroll
            for (uint32_t u = 0; u < U; u++) {
                const uint32_t t = t0 + 32u * u + lane;
                if (t < n_tiles) {
                    R.tcnt[t * (world + 1u) + k] = (uint32_t)(cc + xc[u] - cu[u]);
                    R.tbyt[t * (world + 1u) + k] = cb + xb[u] - bu[u];
                }
                cc += __shfl_sync(0xffffffffu, xc[u], 31);
                cb += __shfl_sync(0xffffffffu, xb[u], 31);
            }
        }
        if (lane == 0) {
            s_tc[k] = cc;
            s_tb[k] = cb;
        }
    }
    __syncthreads();
    if (tid == 0) {
        unsigned long long bc = 0, bb = 0;
        for (uint32_t k = 0; k <= world; k++) {
            R.base[k] = bc;
            R.base[(world + 1u) + k] = bb;
            dest_counts[k] = s_tc[k];
            dest_bytes[k] = s_tb[k];
            if (rx && k < world) {   // the receiver's counts, in its own memory
                rx[k].count[0] = s_tc[k];
                rx[k].count[1] = s_tb[k];
            }
            bc += s_tc[k];
            bb += s_tb[k];
        }
    }
}

// Copy kernels: a warp moves RT_PPW consecutive packets.  Lanes 0..RT_PPW-1
// first gather those packets' metadata and destinations together (two memory
// rounds for all of them instead of two per packet), then the warp copies the
// packets; for each, the first 64 bytes of all RT_PPW packets are loaded before
// any is stored, so short packets need one load round for the whole group.
constexpr uint32_t RT_PPW = 4;

struct RtPkt {
    const uint8_t *src;
    uint8_t *dst;
    uint32_t len;
};

template <bool DISPATCH>
__device__ __forceinline__ void route_copy_group(const RouteWork &R, const uint8_t *in_buf,
                                                 const uint32_t *in_off, const uint16_t *in_len,
                                                 const uint32_t *sa, const uint32_t *sa_map,
                                                 uint32_t n, uint32_t world, uint8_t *send_buf,
                                                 uint16_t *send_len, uint32_t *send_sa,
                                                 const nba_ipsec_peer_rx *rx,
                                                 unsigned long long cap_pkts,
                                                 unsigned long long cap_bytes)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t i0 = w * RT_PPW;
    if (i0 >= n) return;
    // lane q < RT_PPW: packet i0 + q's place
    RtPkt me = {nullptr, nullptr, 0u};
    if (lane < RT_PPW && i0 + lane < n) {
        const uint32_t i = i0 + lane;
        const uint32_t d = R.dest[i];
        const uint32_t len = in_len[i];
        const uint32_t off = in_off[i];
        const uint32_t s = sa[i];
        const uint32_t rk = R.rank[i], brk = R.brank[i];
        if (d < world) {
            const uint32_t tile = i / RT_TILE;
            const unsigned long long pos = R.tcnt[tile * (world + 1u) + d] + rk;
            const unsigned long long boff = R.tbyt[tile * (world + 1u) + d] + brk;
            const uint32_t local = sa_map ? (__ldg(sa_map + s) & 0xFFFFFFu) : s / world;
            if (DISPATCH) {
                if (pos < cap_pkts && boff + len <= cap_bytes) {   // never write out of bounds
                    const nba_ipsec_peer_rx r = rx[d];
                    me = {in_buf + off, r.buf + boff, len};
                    r.off[pos] = (uint32_t)boff;
                    r.len[pos] = (uint16_t)len;
                    r.sa[pos] = local;
                } else if (pos <= cap_pkts && boff <= cap_bytes) {
                    // The receiver's packets that do not fit form a suffix (pos
                    // and boff grow together); this is its FIRST packet, so
                    // exactly this lane publishes the count of what was
                    // written, overriding the scan's totals (the caller sees the
                    // overflow as dest_counts / dest_bytes above rx's count).
                    const nba_ipsec_peer_rx r = rx[d];
                    r.count[0] = pos;
                    r.count[1] = boff;
                }
            } else {
                const unsigned long long gpos = R.base[d] + pos;
                me = {in_buf + off, send_buf + R.base[(world + 1u) + d] + boff, len};
                send_len[gpos] = (uint16_t)len;
                send_sa[gpos] = local;
            }
        }
    }
    RtPkt g[RT_PPW];
#pragma unroll
    for (uint32_t q = 0; q < RT_PPW; q++) {
        g[q].src = reinterpret_cast<const uint8_t *>(
            __shfl_sync(0xffffffffu, reinterpret_cast<unsigned long long>(me.src), q));
        g[q].dst = reinterpret_cast<uint8_t *>(
            __shfl_sync(0xffffffffu, reinterpret_cast<unsigned long long>(me.dst), q));
        g[q].len = __shfl_sync(0xffffffffu, me.len, q);
    }
    // first 64 bytes of every packet: all loads, then all stores
    uint8_t v[RT_PPW][2];
#pragma unroll
    for (uint32_t q = 0; q < RT_PPW; q++) {
        v[q][0] = (g[q].dst && lane < g[q].len) ? g[q].src[lane] : 0;
        v[q][1] = (g[q].dst && lane + 32u < g[q].len) ? g[q].src[lane + 32u] : 0;
    }
#pragma unroll
    for (uint32_t q = 0; q < RT_PPW; q++) {
        if (g[q].dst && lane < g[q].len) g[q].dst[lane] = v[q][0];
        if (g[q].dst && lane + 32u < g[q].len) g[q].dst[lane + 32u] = v[q][1];
    }
    // the rest of longer packets, 16 bytes per lane where source and
    // destination share their alignment, bytes otherwise
#pragma unroll 1
    for (uint32_t q = 0; q < RT_PPW; q++) {
        const uint32_t len = g[q].len;
        if (!g[q].dst || len <= 64u) continue;
        const uint8_t *src = g[q].src;
        uint8_t *dst = g[q].dst;
        const uintptr_t a16 = reinterpret_cast<uintptr_t>(src + 64u) & 15u;
        if (a16 == (reinterpret_cast<uintptr_t>(dst + 64u) & 15u)) {
            const uint32_t head = min(len - 64u, (16u - (uint32_t)a16) & 15u);
            const uint32_t nv = (len - 64u - head) >> 4;
            if (lane < head) dst[64u + lane] = src[64u + lane];
            const uint4 *s4 = reinterpret_cast<const uint4 *>(src + 64u + head);
            uint4 *d4 = reinterpret_cast<uint4 *>(dst + 64u + head);
            for (uint32_t k = lane; k < nv; k += 32u) d4[k] = s4[k];
            for (uint32_t b = 64u + head + 16u * nv + lane; b < len; b += 32u) dst[b] = src[b];
        } else {
            for (uint32_t b = 64u + lane; b < len; b += 32u) dst[b] = src[b];
        }
    }
}

// Bytes to the send buffer (destination-major, batch order inside a
// destination), lengths and local SA indices to the send arrays.
__global__ void __launch_bounds__(256)
k_route_pack(RouteWork R, const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
             const uint32_t *sa, const uint32_t *sa_map, uint32_t n, uint32_t world,
             uint8_t *send_buf, uint16_t *send_len, uint32_t *send_sa)
{
    route_copy_group<false>(R, in_buf, in_off, in_len, sa, sa_map, n, world, send_buf, send_len,
                            send_sa, nullptr, 0ull, 0ull);
}

// Single-ingress dispatch (nba_ipsec_route_dispatch): every packet straight
// into its owner's receive buffers -- own memory or a peer GPU's mapped over
// NVLink -- at the owner-local position (tile prefix + rank within the tile,
// batch order), with its offset, length and local SA index.
__global__ void __launch_bounds__(256)
k_route_dispatch(RouteWork R, const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                 const uint32_t *sa, const uint32_t *sa_map, uint32_t n, uint32_t world,
                 const nba_ipsec_peer_rx *rx, unsigned long long cap_pkts,
                 unsigned long long cap_bytes)
{
    route_copy_group<true>(R, in_buf, in_off, in_len, sa, sa_map, n, world, nullptr, nullptr,
                           nullptr, rx, cap_pkts, cap_bytes);
}

size_t route_workspace_bytes(uint32_t max_pkts, uint32_t world)
{
    const size_t tiles = (max_pkts + RT_TILE - 1) / RT_TILE;
    return 3ull * max_pkts * 4 + tiles * (world + 1) * (4 + 8) + 2ull * (world + 1) * 8 + 256;
}

cudaError_t launch_route(const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                         const uint32_t *sa, uint32_t n, uint32_t n_sa_total,
                         const uint32_t *sa_map, uint32_t world, void *ws, uint8_t *send_buf, uint16_t *send_len, uint32_t *send_sa,
                         unsigned long long *dest_counts, unsigned long long *dest_bytes,
                         cudaStream_t st, const nba_ipsec_peer_rx *rx, unsigned long long cap_pkts,
                         unsigned long long cap_bytes)
{
    const uint32_t tiles = (n + RT_TILE - 1) / RT_TILE;
    uint8_t *p = static_cast<uint8_t *>(ws);
    auto take = [&](size_t b) {
        uint8_t *r = p;
        p += (b + 15) & ~(size_t)15;
        return r;
    };
    RouteWork R;
    R.dest = reinterpret_cast<uint32_t *>(take((size_t)n * 4));
    R.rank = reinterpret_cast<uint32_t *>(take((size_t)n * 4));
    R.brank = reinterpret_cast<uint32_t *>(take((size_t)n * 4));
    R.tcnt = reinterpret_cast<uint32_t *>(take((size_t)tiles * (world + 1) * 4));
    R.tbyt = reinterpret_cast<unsigned long long *>(take((size_t)tiles * (world + 1) * 8));
    R.base = reinterpret_cast<unsigned long long *>(take(2ull * (world + 1) * 8));
    if (tiles) k_route_tiles<<<tiles, RT_TILE, 0, st>>>(R, in_len, sa, n, n_sa_total, sa_map, world);
    k_route_scan<<<1, 32 * (world + 1), 0, st>>>(R, tiles, world, dest_counts, dest_bytes, rx);
    if (n == 0) return cudaGetLastError();
    const uint32_t copy_blocks = ((n + RT_PPW - 1u) / RT_PPW * 32u + 255u) / 256u;   // warp per RT_PPW packets
    if (rx)
        k_route_dispatch<<<copy_blocks, 256, 0, st>>>(R, in_buf, in_off, in_len, sa,
                                                                 sa_map, n, world, rx, cap_pkts,
                                                                 cap_bytes);
    else
        k_route_pack<<<copy_blocks, 256, 0, st>>>(R, in_buf, in_off, in_len, sa, sa_map,
                                                             n, world, send_buf, send_len, send_sa);
    return cudaGetLastError();
}

}  // namespace nba
