// in_replay.cuh -- device helpers of the batch-parallel RFC 4303 §3.4.3
// anti-replay decision (k_in_replay.cu header has the derivation), shared by
// the three-kernel inbound path (k_in_replay / k_in_decide) and the one-kernel
// path (k_in_fused<true>).
#pragma once
#include "internal.cuh"

namespace nba {

__device__ __forceinline__ uint32_t hash_slot(unsigned long long key, uint32_t hmask)
{
    return (uint32_t)((key * 0x9E3779B97F4A7C15ull) >> 32) & hmask;
}

// Max of v over the earlier lanes of this lane's group (lt = the group's lanes
// below this one; 0 when none): one shuffle per earlier group member, the
// loop warp-uniform over the largest such count (a group's lanes share a
// key, so with many SAs a group has one or two lanes per warp) instead of 32
// shuffles.  All 32 lanes call it.
__device__ __forceinline__ uint32_t group_prefix_max(uint32_t lt, uint32_t v)
{
    uint32_t m = lt, mex = 0;
    const uint32_t rounds = __reduce_max_sync(0xffffffffu, (uint32_t)__popc(lt));
    for (uint32_t k = 0; k < rounds; k++) {
        const uint32_t l = m ? (uint32_t)(__ffs(m) - 1) : (threadIdx.x & 31u);
        const uint32_t x = __shfl_sync(0xffffffffu, v, l);
        if (m) mex = max(mex, x);
        m &= m - 1u;
    }
    return mex;
}

// (t0, b0: the SA's window, loaded by the caller beside the row)
__device__ __forceinline__ void window_advance(const InState &S, uint32_t sa, uint32_t batch_max,
                                               uint32_t t0, unsigned long long b0)
{
    S.top_prev[sa] = t0;
    S.bmp_prev[sa] = b0;
    const uint32_t t1 = max(t0, batch_max);
    const uint32_t sh = t1 - t0;
    S.bmp[sa] = sh >= REPLAY_W ? 0ull : (b0 << sh);
    S.top[sa] = t1;
}

// Exclusive prefix max down SA row `sa` of the tile maxima by one warp, then
// the window edge update for the batch.
__device__ __forceinline__ void scan_max_row(const InState &S, uint32_t sa, uint32_t n_tiles,
                                             uint32_t lane)
{
    constexpr int U = 8;
    uint32_t *row = S.hmax + (size_t)sa * n_tiles;
    uint32_t *pfx = S.pmx + (size_t)sa * n_tiles;
    uint32_t carry = 0, w0 = 0;
    unsigned long long b0 = 0;
    if (lane == 0) {                                 // the window, beside the row's loads
        w0 = S.top[sa];
        b0 = S.bmp[sa];
    }
    for (uint32_t t0 = 0; t0 < n_tiles; t0 += 32u * U) {
        uint32_t h[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint32_t t = t0 + 32u * u + lane;
            h[u] = t < n_tiles ? __ldcg(&row[t]) : 0u;
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            if (t0 + 32u * u >= n_tiles) break;
            uint32_t x = h[u];
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= (uint32_t)o) x = max(x, y);
            }
            uint32_t ex = __shfl_up_sync(0xffffffffu, x, 1);
            if (lane == 0) ex = 0;
            const uint32_t t = t0 + 32u * u + lane;
            if (t < n_tiles) {
                pfx[t] = max(carry, ex);
                if (h[u]) row[t] = 0;            // re-arm for the next batch
            }
            carry = max(carry, __shfl_sync(0xffffffffu, x, 31));
        }
    }
    if (lane == 0) window_advance(S, sa, carry, w0, b0);
}

// All SA rows by `nslots` warps (this one is `slot`): one warp per SA for long
// rows, one lane per SA for short ones (small batches, n_tiles <= 32).
__device__ __forceinline__ void scan_all_rows(const InState &S, uint32_t n_sa, uint32_t slot,
                                              uint32_t nslots, uint32_t n_tiles, uint32_t lane)
{
    if (n_tiles > 32u) {
        for (uint32_t sa = slot; sa < n_sa; sa += nslots) scan_max_row(S, sa, n_tiles, lane);
        return;
    }
    for (uint32_t k0 = 0; (size_t)k0 * nslots < n_sa; k0 += 32u) {
        const size_t sa_l = slot + (size_t)(k0 + lane) * nslots;
        if (sa_l >= n_sa) continue;
        const uint32_t sa = (uint32_t)sa_l;
        uint32_t *row = S.hmax + (size_t)sa * n_tiles;
        uint32_t *pfx = S.pmx + (size_t)sa * n_tiles;
        const uint32_t w0 = S.top[sa];
        const unsigned long long b0 = S.bmp[sa];
        uint32_t h[32];
#pragma unroll
        for (uint32_t t = 0; t < 32u; t++) h[t] = t < n_tiles ? __ldcg(&row[t]) : 0u;
        uint32_t carry = 0;
#pragma unroll
        for (uint32_t t = 0; t < 32u; t++) {
            if (t < n_tiles) {
                pfx[t] = carry;
                if (h[t]) row[t] = 0;
            }
            carry = max(carry, h[t]);
        }
        window_advance(S, sa, carry, w0, b0);
    }
}

// The per-packet decision (sequential rule restated for the batch): given the
// window at batch start (t0, b0), the edge seen by the packet (tj = max of t0,
// the earlier tiles' prefix max and the earlier packets of its tile), the
// (sa, q) -> first-index hash of authenticated packets, and the flags of the
// packet.  Accepted packets set their bit in the new window (edge t1).
__device__ __forceinline__ uint32_t replay_decide(const InState &S, uint32_t s, uint32_t i, uint32_t f,
                                                  uint32_t q, uint32_t t0, unsigned long long b0,
                                                  uint32_t tj, uint32_t t1, uint32_t hmask)
{
    bool pass = q != 0u;
    if (pass && q <= tj) {
        if (tj - q >= REPLAY_W) {
            pass = false;                                    // left of the window
        } else if (q <= t0 && ((b0 >> (t0 - q)) & 1ull)) {
            pass = false;                                    // seen before the batch
        } else {                                             // seen earlier in it?
            const unsigned long long k64 = ((unsigned long long)s << 32) | q;
            uint32_t h = hash_slot(k64, hmask);
            while (true) {
                const unsigned long long kk = S.hkey[h];
                if (kk == k64) {
                    if (S.hval[h] < i) pass = false;
                    break;
                }
                if (kk == ~0ull) break;
                h = (h + 1u) & hmask;
            }
        }
    }
    if (!pass) return ST_DROP_REPLAY;
    if (!(f & INF_ICV)) return ST_DROP_AUTH;
    const uint32_t d = t1 - q;                               // new right edge
    if (d < REPLAY_W) atomicOr(&S.bmp[s], 1ull << d);
    return (f & INF_TRL) ? ST_OK : ST_DROP_TRAILER;
}

// (s, q) -> smallest packet index i among the authenticated packets
__device__ __forceinline__ void replay_hash_insert(unsigned long long *hkey, uint32_t *hval, uint32_t s,
                                                   uint32_t q, uint32_t i, uint32_t hmask)
{
    const unsigned long long k64 = ((unsigned long long)s << 32) | q;
    uint32_t h = hash_slot(k64, hmask);
    while (true) {
        const unsigned long long old = atomicCAS(&hkey[h], ~0ull, k64);
        if (old == ~0ull || old == k64) {
            atomicMin(&hval[h], i);
            break;
        }
        h = (h + 1u) & hmask;
    }
}

__device__ __forceinline__ void replay_hash_insert(const InState &S, uint32_t s, uint32_t q, uint32_t i,
                                                   uint32_t hmask)
{
    replay_hash_insert(S.hkey, S.hval, s, q, i, hmask);
}

}  // namespace nba
