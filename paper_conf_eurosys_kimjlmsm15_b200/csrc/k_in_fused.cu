// k_in_fused.cu -- ESP inbound, step 1 of 3: per packet, in
// ONE pass over its bytes, the format checks, the ICV verification and the
// AES-CTR decryption.  The mirror of k_fused.cu (same SM layout: one 512-thread
// CTA per SM, 128 KB bank-replicated T-tables, one lane per packet, length-
// sorted lanes, AES and SHA-1 interleaved every 64 bytes).
//
// RFC 4303 §3.4.4.1 allows the ICV check and the decryption to run in parallel
// as long as the packet is not released before both are done: the plaintext is
// written to the caller's slot here, but out_len stays 0 (= dropped) until
// k_in_decide has combined the ICV result with the anti-replay decision
// (§3.4.3), which needs the authenticated sequence numbers of all earlier
// packets of the SA (k_in_replay).
//
// Per packet i (SA s = sa_idx[i], L = in_len[i], reading B2):
//   format: 72 <= L <= 1552, C = L - 48 = 0 mod 4, outer 0x45, tot_len = L,
//           no fragment, protocol 50, header checksum valid, SPI = spi_s;
//   ICV:    HMAC-SHA1-96 over SPI .. ciphertext (midstates of the SA), compared
//           with the 12 received bytes;
//   decrypt: counter block nonce_s || IV (from the packet, RFC 3686 §3.1) ||
//           BE32(k+1); T = E xor keystream streamed to out_buf + out_off[i];
//   trailer: next header 4, pad length p with D = C - 2 - p >= 20, pad bytes 1..p.
// Output: flags[i] = INF_FMT | INF_ICV | INF_TRL | D, seq[i].
#include "fused_common.cuh"
#include "in_replay.cuh"

namespace nba {

__device__ __forceinline__ uint32_t esp_in_packet(const DevTable &T, const InBatchArgs &B,
                                                  const FusedLo &L, const FusedHi &H,
                                                  uint32_t lane4r, uint32_t tid, uint32_t sa,
                                                  uint32_t C, uint32_t q32, uint32_t iv0,
                                                  uint32_t iv1, uint32_t inoff, uint32_t outoff,
                                                  const uint4 &r0, const uint4 &r1, const uint4 &r2,
                                                  const uint4 &hd, const uint4 &h0, const uint4 &h1)
{
    const uint32_t Cw = C >> 2;                  // ciphertext words
    const uint32_t Mw = 4u + Cw;                 // MAC input words (ESP hdr + ciphertext)
    const uint32_t nsteps = (Cw + 15u) >> 4;     // 64-byte AES steps
    const uint32_t nb_in = (4u * Mw + 8u) / 64u + 1u;   // inner SHA-1 blocks
    const uint32_t bitlen = (64u + 4u * Mw) * 8u;

    const CtrPre cp = ctr_precompute(lane4r, r0, r1, r2, hd.y, iv0, iv1);

    OutStream os;
    os.init(B.out_buf + outoff);
    // SHA-1 message words 0..3 = SPI || seq || IV (big-endian words of the wire bytes)
    uint32_t carry[4] = {bswap32(hd.x), q32, bswap32(iv0), bswap32(iv1)};
    uint32_t st[5] = {h0.x, h0.y, h0.z, h0.w, h1.x};
    const uint8_t *src = B.in_buf + inoff + 36u;          // ciphertext E
    const uintptr_t src_end = reinterpret_cast<uintptr_t>(src) + C;
    if (C > 64u) prefetch_l2(src + 64);
    if (C > 128u) prefetch_l2(src + 128);
    uint32_t lastw = 0, prevw = 0;               // plaintext words Cw-1 and Cw-2

#pragma unroll 1
    for (uint32_t it = 0; it <= nb_in; it++) {
        uint32_t ct[16];
#pragma unroll
        for (int w = 0; w < 16; w++) ct[w] = 0u;
        if (it < nsteps) {
            if (64u * it + 192u < C) prefetch_l2(src + 64u * it + 192u);
            // interior step: the three 32-byte blocks lie inside E and the
            // step holds neither of the last two plaintext words
            const bool interior = 16u * it + 18u <= Cw;
            Raw6 raw;
            if (interior) load_raw6_inb(reinterpret_cast<uintptr_t>(src) + 64u * it, raw);
            else load_raw6(reinterpret_cast<uintptr_t>(src) + 64u * it, src_end, raw);
            uint32_t ks[16];
            aes4_keystream(lane4r, cp, it, L, H, tid, ks);
            extract16(raw, ct);                  // ciphertext words (beyond C: ignored)
            uint32_t pt[16];
#pragma unroll
            for (int w = 0; w < 16; w++) pt[w] = ct[w] ^ ks[w];
            if (!interior) {
                const uint32_t lw = Cw - 1u - 16u * it;
#pragma unroll
                for (int w = 0; w < 16; w++) {
                    if ((uint32_t)w == lw) lastw = pt[w];
                    if ((uint32_t)w + 1u == lw) prevw = pt[w];
                }
            }
            if (16u * it + 16u <= Cw) {
                os.put16(pt);
            } else {
#pragma unroll
                for (int w = 0; w < 16; w++)
                    if (16u * it + w < Cw) os.put(pt[w]);
            }
        }
        // SHA-1 block: inner block `it` over SPI || seq || IV || E (FIPS 180-4
        // §5.1.1 padding), or the outer hash of the inner digest (RFC 2104)
        uint32_t W[16];
        if (it < nb_in) {
            const uint32_t m0 = 16u * it;
            if (m0 + 16u <= Mw) {                     // a block of message words only
#pragma unroll
                for (int i = 0; i < 16; i++) W[i] = i < 4 ? carry[i] : bswap32(ct[i - 4]);
            } else {                                  // FIPS 180-4 §5.1.1 padding
#pragma unroll
                for (int i = 0; i < 16; i++) {
                    const uint32_t m = m0 + i;
                    const uint32_t msg = i < 4 ? carry[i] : bswap32(ct[i - 4]);
                    W[i] = m < Mw ? msg : (m == Mw ? 0x80000000u : 0u);
                }
                if (it == nb_in - 1u) W[15] = bitlen;
            }
#pragma unroll
            for (int i = 0; i < 4; i++) carry[i] = bswap32(ct[12 + i]);
        } else {
#pragma unroll
            for (int i = 0; i < 5; i++) W[i] = st[i];
            W[5] = 0x80000000u;
#pragma unroll
            for (int i = 6; i < 15; i++) W[i] = 0u;
            W[15] = (64u + 20u) * 8u;
            uint4 g4, g5;   // {hout[3], hout[4], -, -}, {hout[0], hout[1], hout[2], 0}
            ldg_nc_v8(&T.sal[(size_t)sa * SAL_U4 + 4], g4, g5);
            st[0] = g5.x; st[1] = g5.y; st[2] = g5.z; st[3] = g4.x; st[4] = g4.y;
        }
        sha1_compress_fma(st, W, T.n_sa != 0u ? 1u : 0u);   // (n_sa >= 1: an opaque 1)
    }
    os.finish(B.out_buf + outoff + C);

    // RFC 4303 §3.4.4.1 / RFC 2404: first 96 bits of the outer digest
    uint32_t icv[3];
    load_words<3>(src_end, src_end + 12u, icv);
    const uint32_t diff = (bswap32(st[0]) ^ icv[0]) | (bswap32(st[1]) ^ icv[1]) |
                          (bswap32(st[2]) ^ icv[2]);
    uint32_t flags = diff == 0u ? INF_ICV : 0u;

    // trailer (reading B4): ... pad 1..p | p | next header, T ends on a word
    const uint32_t nh = lastw >> 24, p = (lastw >> 16) & 0xffu;
    bool trl = nh == 4u && p + 2u + MIN_D <= C;
    if (trl) {
        const uint32_t D = C - 2u - p;
        if (p <= 6u) {               // pad bytes inside the last two words
            const unsigned long long tail = ((unsigned long long)lastw << 32) | prevw;
            for (uint32_t j = 1; j <= p; j++)
                trl &= ((tail >> (8u * (5u - p + j))) & 0xffu) == j;
        } else {                     // long padding: read back this lane's own stores
            const uint8_t *o = B.out_buf + outoff + D;
            for (uint32_t j = 1; j <= p; j++) trl &= o[j - 1] == (uint8_t)j;
        }
        if (trl) flags |= INF_TRL | D;
    }
    return flags;
}

// Format checks of one received packet (reading B2): outer IPv4 header without
// options, total length = L, not a fragment, protocol 50, valid checksum, the
// SA's SPI.  info = C | INFO_OK (0: DROP_FORMAT / DROP_SA), q = the sequence
// number field, iv0 / iv1 = the IV words.
__device__ __forceinline__ void in_format(const DevTable &T, const InBatchArgs &B, uint32_t sa,
                                          uint32_t Lin, uint32_t inoff, uint32_t &info, uint32_t &q,
                                          uint32_t &iv0, uint32_t &iv1)
{
    info = q = iv0 = iv1 = 0;
    if (sa < T.n_sa && Lin >= IN_MIN_LEN && Lin <= IN_MAX_LEN && ((Lin - 48u) & 3u) == 0) {
        const uint8_t *pk = B.in_buf + inoff;
        uint32_t w[9];
        load_words<9>(reinterpret_cast<uintptr_t>(pk), reinterpret_cast<uintptr_t>(pk) + Lin, w);
        // RFC 1071: the one's complement sum over the header (checksum
        // included) is 0xffff; byte order does not matter (§2(B))
        uint32_t sum = 0;
#pragma unroll
        for (int k = 0; k < 5; k++) sum += (w[k] & 0xffffu) + (w[k] >> 16);
        sum = (sum & 0xffffu) + (sum >> 16);
        sum = (sum & 0xffffu) + (sum >> 16);
        const uint32_t tot = ((w[0] >> 8) & 0xff00u) | (w[0] >> 24);
        const bool ok = (w[0] & 0xffu) == 0x45u && tot == Lin &&
                        (w[1] & 0xff3f0000u) == 0u &&         // MF = 0, offset 0
                        ((w[2] >> 8) & 0xffu) == 50u && sum == 0xffffu &&
                        w[5] == __ldg(&T.sahdr[sa]).x;        // SPI (RFC 4303 §3.4.2)
        if (ok) {
            info = (Lin - 48u) | INFO_OK;
            q = bswap32(w[6]);
            iv0 = w[7];
            iv1 = w[8];
        }
    }
}

// ---- one-kernel inbound (n <= F_SUPER x grid): the anti-replay decision of
// k_in_replay / k_in_decide inside this kernel, each CTA one tile of the
// batch (its packets in batch order, thread j <-> packet p_begin + j):
//   tile part: warp-segmented prefix max of the authenticated numbers by SA,
//     merged across the 16 warps through a shared hash; per-SA tile maxima to
//     the SA-major matrix;
//   grid barrier; (sa, q) -> first-index hash inserts; one warp per SA scans
//     its row (exclusive prefix max) and moves the window edge;
//   grid barrier; per-packet decision, window bits, out_len, status, counters.
// The same arithmetic as the three-kernel path (in_replay.cuh), so the same
// result as the sequential receiver.
constexpr uint32_t CTLI_BAR = 4;   // S.ctl word: monotonic barrier arrivals
constexpr uint32_t CTLI_BASE = 5;  // S.ctl word: arrivals before the current one-kernel launch
constexpr uint32_t CTLI_PAR = 6;   // S.ctl word: one-kernel launches so far (hash parity)
constexpr uint32_t CTLI_BAR2 = 7;  // S.ctl word: pipelined ring's row-scan arrivals (monotonic)
#ifndef NBA_IN_LANE_INSERT    // one-kernel inbound: duplicate-hash inserts by the lanes into a
#define NBA_IN_LANE_INSERT 1  //   launch-parity pair of hashes (0: after the first barrier)
#endif

// The one-kernel path's duplicate hashes (S.hk / S.hv by launch parity): the
// lanes insert each authenticated packet into the current one right after
// its ICV check, the tail clears the next launch's one between its two
// barriers (over the whole capacity, `full`).  off: the hash S.hkey / S.hval
// cleared at batch start and filled after the first barrier (plain ring).
struct LaneIns {
    bool on;
    unsigned long long *ck;
    uint32_t *cv;
    unsigned long long *nk;
    uint32_t *nv;
    uint32_t full;
};

__device__ __forceinline__ void in_merged_tail(const DevTable &T, const InState &S0, const InBatchArgs &B,
                                               FusedLo &L, uint8_t *tabs, uint32_t p_begin,
                                               uint32_t p_end, uint32_t hmask, uint32_t bar_base,
                                               const LaneIns &li)
{
    InState S = S0;
    if (li.on) {                                  // the lanes' hash of this launch
        S.hkey = li.ck;
        S.hval = li.cv;
    }
    constexpr uint32_t HS = 2u * F_SUPER, NW = F_THREADS / 32u;
    __shared__ unsigned long long s_cnt[N_IN_COUNTERS - 1];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x, n_sa = T.n_sa;
    const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
    const uint32_t j = tid, i = p_begin + j;
    const bool live = j < cnt;
    const uint32_t f = live ? L.aux1[j] : 0u;
    const uint32_t sa = live ? L.sa[j] : INVALID_SA;
    const uint32_t q = (f & INF_FMT) ? L.seq[j] : 0u;
    const uint32_t key = (f & INF_FMT) ? sa : INVALID_SA;
    const bool inA = (f & INF_ICV) != 0u;
    const uint32_t qa = inA ? q : 0u;
    for (uint32_t k = tid; k < HS; k += F_THREADS) {
        L.hkey[k] = INVALID_SA;
        L.hmask[k] = 0;
    }
    if (tid < N_IN_COUNTERS - 1) s_cnt[tid] = 0;
    // per-warp group maxima, [HS][NW] u32 = 64 KB in the (now unused) T-tables
    uint32_t(*gm)[NW] = reinterpret_cast<uint32_t(*)[NW]>(tabs);
    const uint32_t peers = __match_any_sync(0xffffffffu, key);
    const uint32_t lt = peers & lanemask_lt();
    const uint32_t mex = group_prefix_max(lt, qa);   // max over earlier lanes of the group
    const uint32_t leader = __ffs(peers) - 1, hi_lane = 31u - __clz(peers);
    const uint32_t gmax = __shfl_sync(0xffffffffu, max(mex, qa), hi_lane);
    __syncthreads();   // CTA hash initialised, T-tables no longer read
    uint32_t slot = 0;
    if (key != INVALID_SA && lane == leader) {
        slot = (key * 0x9E3779B1u) >> 22;           // 10 bits -> HS = 1024 slots
        while (true) {
            const uint32_t old = atomicCAS(&L.hkey[slot], INVALID_SA, key);
            if (old == INVALID_SA || old == key) break;
            slot = (slot + 1u) & (HS - 1u);
        }
        gm[slot][warp] = gmax;
        atomicOr(&L.hmask[slot], 1u << warp);
    }
    slot = __shfl_sync(0xffffffffu, slot, leader);
    __syncthreads();
    uint32_t base = 0;
    if (key != INVALID_SA) {
        const uint32_t m = L.hmask[slot];
#pragma unroll
        for (uint32_t w = 0; w < NW; w++)
            if (w < warp && ((m >> w) & 1u)) base = max(base, gm[slot][w]);
        const uint32_t tmax = max(base, gmax);       // per-tile SA maximum, nonzero only
        if ((m >> (warp + 1u)) == 0u && lane == hi_lane && tmax != 0u)
            S.hmax[(size_t)key * G + cta] = tmax;
    }
    const uint32_t lmax = max(base, mex);
    __syncthreads();
    grid_arrive(&S.ctl[CTLI_BAR]);
    grid_wait(&S.ctl[CTLI_BAR], bar_base + G);
    // every CTA has read the base and the parity (before arriving): advance
    // them for the next launch
    if (cta == 0 && tid == 0) {
        S.ctl[CTLI_BASE] = bar_base + 2u * G;
        if (li.on) S.ctl[CTLI_PAR] = S.ctl[CTLI_PAR] + 1u;
    }
    scan_all_rows(S, n_sa, warp * G + cta, G * NW, G, lane);   // SA s on CTA s mod G
    if (li.on) {
        // the next launch's hash, cleared before this launch's second barrier
        // (its previous user, the launch before this one, has completed)
        for (uint32_t k = cta * F_THREADS + tid; k <= li.full; k += G * F_THREADS) {
            li.nk[k] = ~0ull;
            li.nv[k] = ~0u;
        }
    } else if (inA) {
        replay_hash_insert(S, key, q, i, hmask);  // (the hash was cleared before the barrier)
    }
    __syncthreads();
    grid_arrive(&S.ctl[CTLI_BAR]);
    grid_wait(&S.ctl[CTLI_BAR], bar_base + 2u * G);
    uint32_t st = 0xffu, D = 0, Lin = 0;
    if (live) {
        if (sa >= n_sa) {
            st = ST_DROP_SA;
        } else if (!(f & INF_FMT)) {
            st = ST_DROP_FORMAT;
        } else {
            const uint32_t t0 = S.top_prev[sa];
            const unsigned long long b0 = S.bmp_prev[sa];
            const uint32_t tj = max(t0, max(S.pmx[(size_t)sa * G + cta], lmax));
            st = replay_decide(S, sa, i, f, q, t0, b0, tj, S.top[sa], hmask);
            if (st == ST_OK) {
                D = f & 0xffffu;
                Lin = B.in_len[i];
            }
        }
        B.out_len[i] = (uint16_t)D;
        if (B.status) B.status[i] = (uint8_t)st;
    }
    // counters: pkts_ok, drop_sa, drop_format, drop_replay, drop_auth,
    // drop_trailer, bytes_in, bytes_out (+ batches by CTA 0)
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
    if (tid == 0 && cta == 0) atomicAdd(&S.counters[N_IN_COUNTERS - 1], 1ull);
}

// One batch (the body of k_in_fused; k_in_fused_ring runs it for a sequence
// of batches).  bar_base: the batch's grid-barrier base (one-kernel form).
template <bool MERGED>
__device__ __forceinline__ void in_fused_body(const DevTable &T, const InState &S,
                                              const InBatchArgs &B, uint32_t ppc, uint32_t hmask,
                                              uint32_t bar_base, bool tinit, uint32_t tphase,
                                              const LaneIns &li)
{
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t n_sa = T.n_sa;

    const uint32_t sb = smem_u32(smem);
    const uint32_t toff = (0x10000u - (sb & 0xffffu)) & 0xffffu;
    uint32_t lo_off = 0;
    if (toff < sizeof(FusedLo)) {
        if (toff + AES_TABLE_BYTES + sizeof(FusedHi) + sizeof(FusedLo) > F_SMEM) __trap();
        lo_off = toff + AES_TABLE_BYTES + (uint32_t)sizeof(FusedHi);
    }
    uint8_t *tabs = smem + toff;
    FusedLo &L = *reinterpret_cast<FusedLo *>(smem + lo_off);
    FusedHi &H = *reinterpret_cast<FusedHi *>(smem + toff + AES_TABLE_BYTES);
    const uint32_t lane4r = (lane * 4u) | (smem_u32(tabs) & 0xffff0000u);

    // this batch's duplicate-detection hash (read by k_in_replay / k_in_decide
    // of this batch only; the previous batch's kernels have completed) -- with
    // lane inserts the previous launch cleared it
    if (!li.on) {
        for (uint32_t k = blockIdx.x * blockDim.x + tid; k <= hmask; k += gridDim.x * blockDim.x) {
            S.hkey[k] = ~0ull;
            S.hval[k] = ~0u;
        }
    }
    // T-tables by bulk copy (re-staged per batch: the replay merge of the
    // previous batch used their shared memory as scratch); waited for (phase
    // tphase of the mbarrier) before the first lookup
    tables_stage(tabs, T, &L.tbar, tinit);
    if (tid < NBINS) L.bins[tid] = 0;
    __syncthreads();

    const uint32_t p_begin = blockIdx.x * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    for (uint32_t base = p_begin; base < p_end; base += F_SUPER) {
        const uint32_t cnt_pk = min((uint32_t)F_SUPER, p_end - base);
        // ---- 1. metadata and format checks (thread j <-> packet base + j) ----
        const uint32_t j = tid;
        const uint32_t i = base + j;
        if (j < cnt_pk) {
            const uint32_t sa = B.sa_idx[i];
            const uint32_t Lin = B.in_len[i];
            const uint32_t inoff = B.in_off[i];
            uint32_t info = 0, q = 0, iv0 = 0, iv1 = 0;
            in_format(T, B, sa, Lin, inoff, info, q, iv0, iv1);
            L.sa[j] = sa;
            L.info[j] = info;
            L.seq[j] = q;
            L.inoff[j] = inoff;
            L.outoff[j] = B.out_off[i];
            L.aux0[j] = iv0;
            L.aux1[j] = iv1;
        }
        const uint32_t bin_j = (j < cnt_pk && L.info[j]) ? hmac_bin(true, L.info[j] & 0xffffu) : NBINS - 1;
        warp_agg_add(L.bins, bin_j, j < cnt_pk);
        length_sort(L, j, cnt_pk, bin_j);

        // ---- 2. one lane per packet, runs of length-sorted packets placed on
        //         warps by length_sort (LPT over the SM sub-partitions) ----
        {
            uint32_t pos;
            const bool have = lane_position(L, cnt_pk, pos);
            const uint32_t pk = have ? L.perm[pos] : 0u;
            const uint32_t info = have ? L.info[pk] : 0u;
            const uint32_t sa_me = (info & INFO_OK) ? L.sa[pk] : INVALID_SA;
            if (have) {
                uint32_t flags = 0;
                if (info & INFO_OK) {
                    // the SA line (AES key, header words, inner midstate); round
                    // keys 1..10 expanded in the lane
                    uint4 r0, hd, h0, h1, r1, r2;
                    const uint4 *line = T.sal + (size_t)sa_me * SAL_U4;
                    ldg_nc_v8(&line[0], r0, hd);
                    ldg_nc_v8(&line[2], h0, h1);
                    tables_bulk_wait(&L.tbar, tphase);
                    expand_key_lane(lane4r, r0, r1, r2, L, H, tid);
                    flags = INF_FMT | esp_in_packet(T, B, L, H, lane4r, tid, sa_me, info & 0xffffu,
                                                    L.seq[pk], L.aux0[pk], L.aux1[pk], L.inoff[pk],
                                                    L.outoff[pk], r0, r1, r2, hd, h0, h1);
                }
                if (MERGED) {
                    L.aux1[pk] = flags;                 // for the in-kernel replay decision
                    if (li.on && (flags & INF_ICV))     // (sa, q) -> first index, now
                        replay_hash_insert(li.ck, li.cv, sa_me, L.seq[pk], base + pk, hmask);
                } else {
                    S.flags[base + pk] = flags;
                    S.seq[base + pk] = L.seq[pk];
                }
            }
        }
        __syncthreads();
    }
    // every thread has seen the bulk copy land (also those without packets):
    // the tail uses the table region as scratch, and no copy may be in flight
    // when the CTA exits
    tables_bulk_wait(&L.tbar, tphase);
    if constexpr (MERGED) in_merged_tail(T, S, B, L, tabs, p_begin, p_end, hmask, bar_base, li);
}

template <bool MERGED>
__global__ void __launch_bounds__(F_THREADS, 1)
k_in_fused(DevTable T, InState S, InHashPair HP, InBatchArgs B, uint32_t ppc, uint32_t hmask,
           uint32_t hfull, uint32_t bar_base_h)
{
    // one-kernel form: the barrier base and the hash parity live on the device
    // (launches carry no host state and can be recorded in a graph); read
    // before arriving
    const uint32_t bar_base =
        MERGED ? *reinterpret_cast<volatile uint32_t *>(&S.ctl[CTLI_BASE]) : bar_base_h;
    LaneIns li{false, nullptr, nullptr, nullptr, nullptr, 0u};
    if (MERGED && NBA_IN_LANE_INSERT) {
        const uint32_t par = *reinterpret_cast<volatile uint32_t *>(&S.ctl[CTLI_PAR]) & 1u;
        li = par ? LaneIns{true, HP.hk[1], HP.hv[1], HP.hk[0], HP.hv[0], hfull}
                 : LaneIns{true, HP.hk[0], HP.hv[0], HP.hk[1], HP.hv[1], hfull};
    }
    in_fused_body<MERGED>(T, S, B, ppc, hmask, bar_base, true, 0u, li);
}

// An inbound batch ring as ONE persistent launch: the grid walks the run's
// batches (two grid barriers each).  The duplicate-detection hash alternates
// between two buffers by batch parity: batch bi + 1 clears its buffer while
// slower CTAs may still read batch bi's, and batch bi - 1 (the buffer's last
// user) finished everywhere before batch bi's first barrier.  The T-tables are
// re-staged per batch (the replay merge uses their shared memory as scratch).
__global__ void __launch_bounds__(F_THREADS, 1)
k_in_fused_ring(DevTable T, InState S, const InBatchArgs *slots, RingRun R, uint32_t hmask,
                unsigned long long *hkey_b, uint32_t *hval_b)
{
    const uint32_t n_slots = R.n_slots, n_batches = R.n_batches;
    if (R.ts && blockIdx.x == 0 && threadIdx.x == 0) R.ts[0] = gtimer();
    const uint32_t base0 = *reinterpret_cast<volatile uint32_t *>(&S.ctl[CTLI_BASE]);
    const uint32_t G = gridDim.x;
    for (uint32_t bi = 0; bi < n_batches; bi++) {
        const InBatchArgs B = slots[(R.first + bi) % n_slots];
        InState Sb = S;
        if (bi & 1u) {
            Sb.hkey = hkey_b;
            Sb.hval = hval_b;
        }
        uint32_t ppc = (B.n + G - 1) / G;
        ppc = (ppc + 31u) & ~31u;
        if (ppc < 32u) ppc = 32u;
        in_fused_body<true>(T, Sb, B, ppc, hmask, base0 + 2u * bi * G, bi == 0, bi & 1u,
                            LaneIns{false, nullptr, nullptr, nullptr, nullptr, 0u});
        __syncthreads();   // shared memory is reused by the next batch
        if (R.ts && threadIdx.x == 0) atomicMax(&R.ts[1u + bi], gtimer());
    }
}

// ------------------------------------------ software-pipelined inbound ring
// k_in_fused_ring_pipe: the inbound ring with warp roles, as the outbound
// k_fused_ring_pipe.  Per batch k: warps 0..13 ("lanes") take their packet's
// fields (named barrier 2) and run the ICV check + decryption, leaving each
// packet's flags and sequence number in L.tailf / L.tailq (by packet index);
// warps 14..15 meanwhile prepare batch k + 1 -- metadata, format checks (the
// outer header of every packet), length order and LPT run placement -- so
// neither the metadata's DRAM latency nor the header loads sit on the
// critical path; then the whole CTA runs batch k's anti-replay tail (the
// same arithmetic as in_merged_tail: warp-segmented prefix maxima, the CTA's
// SA hash, the (SA, CTA) tile maxima, grid barrier, first-index hash inserts
// and row scans, grid barrier, decisions).  The per-warp group maxima of the
// tail live in the lanes' round-key slots (L.rkA / H.rkB, free once the lanes
// are done), so the T-tables stay in shared memory for the whole run (staged
// once).  The duplicate hash alternates between two buffers by batch parity;
// batch k clears its buffer before its first barrier, and that buffer's last
// user (batch k - 2) finished everywhere before batch k - 1's second barrier.

#ifndef NBA_IN_LANE_FORMAT    // pipelined inbound ring: the outer-header format checks by the
#define NBA_IN_LANE_FORMAT 0  //   lanes (1) or by the side warps' prologue (0)
#endif
#ifndef NBA_IN_PREFETCH       // pipelined inbound ring: L2 prefetches of the next batch's headers
#define NBA_IN_PREFETCH 0     //   and the one after's metadata, ahead of the side warps' prologue
#endif
#ifndef NBA_IN_LANE_ROWS      // pipelined inbound ring: the previous batch's row scans by the
#define NBA_IN_LANE_ROWS 0    //   lane warps at the start of the iteration (1) or the side warps (0)
#endif
#ifndef NBA_IN_PRO_FIRST      // pipelined inbound ring: the side warps run the next batch's
#define NBA_IN_PRO_FIRST 0    //   prologue before (1) or after (0) the previous batch's row scans
#endif
#ifndef NBA_RING_TRACE        // debug variant: per-(batch, CTA) phase stamps into RingRun::ts
#define NBA_RING_TRACE 0
#endif
#if NBA_RING_TRACE
#define IRTR(bi, k) (R.ts ? R.ts + ((size_t)(bi) * gridDim.x + blockIdx.x) * 16u + (k) : nullptr)
#endif

// Prefetches for the side warps' prologue, so its loads hit L2: the CTA's
// range of a batch's metadata arrays (a batch ahead), and -- from the offsets,
// then in L2 -- the outer headers of its packets (at the start of the
// iteration before the prologue, ahead of the row scans).
__device__ __forceinline__ void in_pipe_prefetch_meta(const InBatchArgs &B, uint32_t ppc, uint32_t pt)
{
    const uint32_t p_begin = blockIdx.x * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    if (p_end <= p_begin) return;
    auto lines = [&](const void *base, uint32_t esz) {
        const uintptr_t a = reinterpret_cast<uintptr_t>(base) + (uintptr_t)p_begin * esz;
        const uintptr_t e = reinterpret_cast<uintptr_t>(base) + (uintptr_t)p_end * esz;
        for (uintptr_t x = (a & ~(uintptr_t)127) + 128u * pt; x < e; x += 128u * PIPE_P)
            prefetch_l2(reinterpret_cast<const void *>(x));
    };
    lines(B.sa_idx, 4u);
    lines(B.in_len, 2u);
    lines(B.in_off, 4u);
    lines(B.out_off, 4u);
}

__device__ __forceinline__ void in_pipe_prefetch_hdr(const InBatchArgs &B, uint32_t ppc, uint32_t pt)
{
    constexpr uint32_t PR = PIPE_MAX_PPC / PIPE_P;
    const uint32_t p_begin = blockIdx.x * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
    uint32_t off[PR];
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {
        const uint32_t j = r * PIPE_P + pt;
        off[r] = j < cnt ? B.in_off[p_begin + j] : 0u;
    }
#pragma unroll
    for (uint32_t r = 0; r < PR; r++)
        if (r * PIPE_P + pt < cnt) prefetch_l2(B.in_buf + off[r]);
}

// Metadata + format checks + length order of one inbound batch by the 64
// prologue threads (pt = 0..63) of this CTA.
__device__ __forceinline__ void in_pipe_prologue(const DevTable &T, const InBatchArgs &B, uint32_t ppc,
                                                 FusedLo &L, uint32_t pt, unsigned long long *tr = nullptr)
{
    constexpr uint32_t PR = PIPE_MAX_PPC / PIPE_P;                  // 7 rounds
    const uint32_t lane = pt & 31u, pw = pt >> 5;
    const uint32_t p_begin = blockIdx.x * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
    const uint32_t rounds = (cnt + PIPE_P - 1u) / PIPE_P;
    uint32_t mS[PR], mL[PR], mI[PR], mO[PR];
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {                             // all loads issued together
        const uint32_t j = r * PIPE_P + pt, i = p_begin + j;
        mS[r] = j < cnt ? B.sa_idx[i] : INVALID_SA;
        mL[r] = j < cnt ? B.in_len[i] : 0u;
        mI[r] = j < cnt ? B.in_off[i] : 0u;
        mO[r] = j < cnt ? B.out_off[i] : 0u;
    }
#pragma unroll
    for (uint32_t r = 0; r < PR; r++)                               // outer headers -> L2 / L1
        if (r * PIPE_P + pt < cnt) prefetch_l2(B.in_buf + mI[r]);
    // format checks, the header loads of several rounds in flight together
    // (no shared-memory side effects in between), then the stores
    // (NBA_IN_LANE_FORMAT: the lanes check the format themselves; here the
    // payload length the length order and the LPT costs use, and the outer
    // length in place of the sequence number)
    uint32_t mF[PR], mQ[PR], mV0[PR], mV1[PR];
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {
        mF[r] = mQ[r] = mV0[r] = mV1[r] = 0u;
        if (NBA_IN_LANE_FORMAT) {
            const uint32_t Lin = mL[r];
            if (mS[r] < T.n_sa && Lin >= IN_MIN_LEN && Lin <= IN_MAX_LEN && ((Lin - 48u) & 3u) == 0)
                mF[r] = (Lin - 48u) | INFO_OK;
            mQ[r] = Lin;
        } else if (r * PIPE_P + pt < cnt) {
            in_format(T, B, mS[r], mL[r], mI[r], mF[r], mQ[r], mV0[r], mV1[r]);
        }
    }
    if (tr && pt == 0) tr[10] = gtimer();
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {                             // (unrolled: arrays in registers)
        if (r >= rounds) break;
        const uint32_t j = r * PIPE_P + pt;
        uint32_t bin = NBINS - 1;
        if (j < cnt) {
            L.sa[j] = mS[r];
            L.info[j] = mF[r];
            L.seq[j] = mQ[r];
            L.inoff[j] = mI[r];
            L.outoff[j] = mO[r];
            L.aux0[j] = mV0[r];
            L.aux1[j] = mV1[r];
            if (mF[r]) bin = hmac_bin(true, mF[r] & 0xffffu);
        }
        warp_agg_add(L.bins, bin, j < cnt);
    }
    bar_sync_n(1, PIPE_P);
    if (tr && pt == 0) tr[11] = gtimer();
    bool one_bin = false;
    if (pw == 0) {                                                  // bins -> cursors
        const uint32_t cb = L.bins[lane];
        one_bin = __any_sync(0xffffffffu, cb == cnt);
        uint32_t x = cb;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= (uint32_t)o) x += y;
        }
        L.bins[lane] = x - cb;
        if (lane == 0) L.pstat[2] = one_bin ? 4u : 0u;
    }
    bar_sync_n(1, PIPE_P);
    one_bin = (L.pstat[2] & 4u) != 0u;
    for (uint32_t r = 0; r < rounds; r++) {
        const uint32_t j = r * PIPE_P + pt;
        if (one_bin) {                           // counting sort of one bin = index order
            if (j < cnt) L.perm[j] = (uint16_t)j;
            continue;
        }
        const uint32_t info = j < cnt ? L.info[j] : 0u;
        const uint32_t bin = info ? hmac_bin(true, info & 0xffffu) : NBINS - 1;
        const uint32_t pos = warp_agg_add(L.bins, bin, j < cnt);
        if (j < cnt) L.perm[pos] = (uint16_t)j;
    }
    bar_sync_n(1, PIPE_P);
    if (tr && pt == 0) tr[12] = gtimer();
    if (pt < NBINS) L.bins[pt] = 0u;
    if (pw == 0) {
        // runs of 32 sorted positions -> lane warps, longest first onto the
        // least loaded sub-partition (as the outbound pipelined ring)
        const uint32_t nruns = (cnt + 31u) / 32u;
        uint32_t cost = 0;
        if (lane < nruns) {
            const uint32_t info = L.info[L.perm[32u * lane]];
            const uint32_t C = info & 0xffffu;
            cost = info ? 8u * (esp_nsha_inner(C) + 1u) + 3u * ((C + 15u) >> 4) : 1u;
        }
        const uint32_t c0 = __shfl_sync(0xffffffffu, cost, 0);
        uint32_t mine = lane < nruns ? lane : 0xffu;
        if (!__all_sync(0xffffffffu, lane >= nruns || cost == c0))
            mine = lpt_place(cost, nruns, lane, 4u, 4u, 3u, 3u);
        if (lane < PIPE_LANE_WARPS) L.wrun[lane] = (uint8_t)mine;
    }
}

// Batch k's tile part by the whole CTA (thread j <-> packet p_begin + j), the
// first half of in_merged_tail: warp-segmented prefix maxima of the
// authenticated sequence numbers per SA, the CTA's SA hash, the (SA, CTA)
// tile maxima into S.hmax; each packet's decision inputs (flags, number,
// prefix max within the CTA, SA) go to the CTA's scratch row, and the CTA
// arrives at the batch's first barrier (SB1) without waiting for it.  The
// per-warp group maxima live in the lanes' round-key slots (L.rkA / H.rkB,
// free once the lanes are done), so the T-tables stay in shared memory.
__device__ __forceinline__ void in_pipe_tile(const InState &S, FusedLo &L, FusedHi &H, uint32_t cnt,
                                             uint4 *scr)
{
    constexpr uint32_t HS = 2u * F_SUPER, NW = F_THREADS / 32u;
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x;
    const uint32_t j = tid;
    const bool live = j < cnt;
    const uint32_t f = live ? L.tailf[j] : 0u;
    const uint32_t sa = live ? L.tails[j] : INVALID_SA;
    const uint32_t q = (f & INF_FMT) ? L.tailq[j] : 0u;
    const uint32_t key = (f & INF_FMT) ? sa : INVALID_SA;
    const uint32_t qa = (f & INF_ICV) ? q : 0u;
    for (uint32_t k = tid; k < HS; k += F_THREADS) {
        L.hkey[k] = INVALID_SA;
        L.hmask[k] = 0;
    }
    // per-warp group maxima [HS][NW] u32: slots < 512 in L.rkA, the rest in H.rkB
    auto gm = [&](uint32_t slot) -> uint32_t * {
        uint32_t *b = slot < 512u ? reinterpret_cast<uint32_t *>(&L.rkA[0][0])
                                  : reinterpret_cast<uint32_t *>(&H.rkB[0][0]);
        return b + (slot & 511u) * NW;
    };
    const uint32_t peers = __match_any_sync(0xffffffffu, key);
    const uint32_t lt = peers & lanemask_lt();
    const uint32_t mex = group_prefix_max(lt, qa);   // max over earlier lanes of the group
    const uint32_t leader = __ffs(peers) - 1, hi_lane = 31u - __clz(peers);
    const uint32_t gmax = __shfl_sync(0xffffffffu, max(mex, qa), hi_lane);
    __syncthreads();   // CTA hash initialised, round-key slots no longer read
    uint32_t slot = 0;
    if (key != INVALID_SA && lane == leader) {
        slot = (key * 0x9E3779B1u) >> 22;           // 10 bits -> HS = 1024 slots
        while (true) {
            const uint32_t old = atomicCAS(&L.hkey[slot], INVALID_SA, key);
            if (old == INVALID_SA || old == key) break;
            slot = (slot + 1u) & (HS - 1u);
        }
        gm(slot)[warp] = gmax;
        atomicOr(&L.hmask[slot], 1u << warp);
    }
    slot = __shfl_sync(0xffffffffu, slot, leader);
    __syncthreads();
    uint32_t base = 0;
    if (key != INVALID_SA) {
        const uint32_t m = L.hmask[slot];
        const uint32_t *g = gm(slot);
#pragma unroll
        for (uint32_t w = 0; w < NW; w++)
            if (w < warp && ((m >> w) & 1u)) base = max(base, g[w]);
        const uint32_t tmax = max(base, gmax);       // per-tile SA maximum, nonzero only
        if ((m >> (warp + 1u)) == 0u && lane == hi_lane && tmax != 0u)
            S.hmax[(size_t)key * G + cta] = tmax;
    }
    if (live) scr[j] = make_uint4(f, q, max(base, mex), sa);
    __syncthreads();
    grid_arrive(&S.ctl[CTLI_BAR]);
}

// Side-warp grid barrier: only the 64 prologue threads of each CTA wait.
__device__ __forceinline__ void side_wait(const uint32_t *count, uint32_t target, uint32_t pt)
{
    if (pt == 0) {
        uint32_t v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(count) : "memory");
        } while ((int)(v - target) < 0);
    }
    bar_sync_n(1, PIPE_P);
}

// Row scans of SA rows sa0, sa0 + stride, ... by one warp, RW rows at a time
// with every load of the RW rows issued first; n_tiles <= 160, lane l holding
// tiles 5 l .. 5 l + 4 (a running max in registers, one warp scan of the lane
// maxima).  The arithmetic of scan_max_row.
__device__ __forceinline__ void scan_rows_batched(const InState &S, uint32_t sa0, uint32_t stride,
                                                  uint32_t n_sa, uint32_t n_tiles, uint32_t lane)
{
    constexpr int RW = 4, U = 5;
    for (uint32_t b = sa0; b < n_sa; b += RW * stride) {
        uint32_t h[RW][U], w0[RW];
        unsigned long long b0[RW];
#pragma unroll
        for (int r = 0; r < RW; r++) {
            const uint32_t sa = b + r * stride;
            const bool ok = sa < n_sa;
#pragma unroll
            for (int u = 0; u < U; u++) {
                const uint32_t t = U * lane + u;
                h[r][u] = ok && t < n_tiles ? __ldcg(&S.hmax[(size_t)sa * n_tiles + t]) : 0u;
            }
            w0[r] = ok && lane == 0 ? S.top[sa] : 0u;
            b0[r] = ok && lane == 0 ? S.bmp[sa] : 0ull;
        }
#pragma unroll
        for (int r = 0; r < RW; r++) {
            const uint32_t sa = b + r * stride;
            if (sa >= n_sa) break;
            uint32_t lm = 0;                                       // this lane's tiles' max
#pragma unroll
            for (int u = 0; u < U; u++) lm = max(lm, h[r][u]);
            uint32_t x = lm;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= (uint32_t)o) x = max(x, y);
            }
            uint32_t run = __shfl_up_sync(0xffffffffu, x, 1);      // max over the earlier lanes
            if (lane == 0) run = 0;
            const uint32_t carry = __shfl_sync(0xffffffffu, x, 31);
#pragma unroll
            for (int u = 0; u < U; u++) {
                const uint32_t t = U * lane + u;
                if (t < n_tiles) {
                    S.pmx[(size_t)sa * n_tiles + t] = run;
                    if (h[r][u]) S.hmax[(size_t)sa * n_tiles + t] = 0;   // re-arm
                }
                run = max(run, h[r][u]);
            }
            if (lane == 0) window_advance(S, sa, carry, w0[r], b0[r]);
        }
    }
}

// Batch k's replay, second half, part 1 by the 64 side threads of the CTA
// while the lanes run batch k + 1: wait for every CTA's tile part (SB1 =
// sb1), this CTA's share of the SA row scans (prefix maxima down each
// (SA, CTA) row, window edge update), arrival at SB2 (its own counter,
// CTLI_BAR2: a CTA with no packets in batch k does not wait for SB2, so its
// next tile arrival must not count towards it), and this CTA's slice of the
// duplicate hash clr (batch k + 3's) cleared.
__device__ __forceinline__ void in_pipe_rows(const DevTable &T, const InState &S, uint32_t hmask,
                                             uint32_t sb1, unsigned long long *clr_k, uint32_t *clr_v,
                                             uint32_t pt, unsigned long long *tr)
{
    const uint32_t lane = pt & 31u, pw = pt >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x;
    side_wait(&S.ctl[CTLI_BAR], sb1, pt);
    if (tr && pt == 0) tr[1] = gtimer();
    scan_rows_batched(S, pw * G + cta, 2u * G, T.n_sa, G, lane);
    bar_sync_n(1, PIPE_P);                           // (orders both warps' stores before the arrival)
    if (pt == 0) asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&S.ctl[CTLI_BAR2]) : "memory");
    if (tr && pt == 0) tr[8] = gtimer();
    if (clr_k)
        for (uint32_t k = cta * PIPE_P + pt; k <= hmask; k += G * PIPE_P) {
            clr_k[k] = ~0ull;
            clr_v[k] = ~0u;
        }
}

// The same by the 14 lane warps (NBA_IN_LANE_ROWS), at the start of batch
// k + 1's iteration once they took their fields: wait for SB1 (one thread,
// then named barrier 3 over the 448 lane threads), one SA row per warp at
// most (SA s on CTA s mod G, warp s / G), batch k + 3's hash slice cleared,
// arrival at SB2 once every lane warp's stores are ordered.
__device__ __forceinline__ void in_pipe_rows_lanes(const DevTable &T, const InState &S, uint32_t hmask,
                                                   uint32_t sb1, unsigned long long *clr_k, uint32_t *clr_v,
                                                   unsigned long long *tr)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x;
    if (tid == 0) {
        uint32_t v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&S.ctl[CTLI_BAR]) : "memory");
        } while ((int)(v - sb1) < 0);
        if (tr) tr[1] = gtimer();
    }
    bar_sync_n(3, PIPE_MAX_PPC);
    scan_rows_batched(S, warp * G + cta, PIPE_LANE_WARPS * G, T.n_sa, G, lane);
    if (clr_k)
        for (uint32_t k = cta * PIPE_MAX_PPC + tid; k <= hmask; k += G * PIPE_MAX_PPC) {
            clr_k[k] = ~0ull;
            clr_v[k] = ~0u;
        }
    bar_sync_n(3, PIPE_MAX_PPC);                 // (orders every lane warp's stores before the arrival)
    if (tid == 0) {
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&S.ctl[CTLI_BAR2]) : "memory");
        if (tr) tr[8] = gtimer();
    }
}

// Part 2, by one warp for packets j = 32 w + lane of the CTA's batch-k range
// (w: the warp's slot, 0..13 -- the lane warps once their own packets are
// done): wait for SB2 (every row scanned, sb2), then the decisions:
// statuses, lengths, counters into the CTA's shared counters.
__device__ __forceinline__ void in_pipe_decide(const DevTable &T, const InState &S, const InBatchArgs &B,
                                               uint32_t ppc, const uint4 *scr, uint32_t hmask,
                                               const unsigned long long *hk, const uint32_t *hv,
                                               uint32_t sb2, uint32_t w, unsigned long long *s_cnt)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t G = gridDim.x, cta = blockIdx.x, n_sa = T.n_sa;
    const uint32_t p_begin = cta * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
    if (32u * w >= cnt) return;
    if (lane == 0) {
        uint32_t v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&S.ctl[CTLI_BAR2]) : "memory");
        } while ((int)(v - sb2) < 0);
    }
    __syncwarp();
    const uint32_t j = 32u * w + lane, i = p_begin + j;
    uint32_t st = 0xffu, D = 0, Lin = 0;
    if (j < cnt) {
        const uint4 d = scr[j];
        const uint32_t f = d.x, q = d.y, sa = d.w;
        if (sa >= n_sa) {
            st = ST_DROP_SA;
        } else if (!(f & INF_FMT)) {
            st = ST_DROP_FORMAT;
        } else {
            const uint32_t t0 = __ldcg(&S.top_prev[sa]);
            const unsigned long long b0 = __ldcg(&S.bmp_prev[sa]);
            const uint32_t pm = __ldcg(&S.pmx[(size_t)sa * G + cta]);
            const uint32_t t1 = __ldcg(&S.top[sa]);
            InState Sd = S;
            Sd.hkey = const_cast<unsigned long long *>(hk);
            Sd.hval = const_cast<uint32_t *>(hv);
            st = replay_decide(Sd, sa, i, f, q, t0, b0, max(t0, max(pm, d.z)), t1, hmask);
            if (st == ST_OK) {
                D = f & 0xffffu;
                Lin = B.in_len[i];
            }
        }
        B.out_len[i] = (uint16_t)D;
        if (B.status) B.status[i] = (uint8_t)st;
    }
    // counters: pkts_ok, drop_sa, drop_format, drop_replay, drop_auth,
    // drop_trailer, bytes_in, bytes_out (warp sums into the CTA's counters)
#pragma unroll
    for (uint32_t k = 0; k < 6; k++) {
        const uint32_t x = __reduce_add_sync(0xffffffffu, st == k ? 1u : 0u);
        if (lane == 0 && x) atomicAdd(&s_cnt[k], (unsigned long long)x);
    }
    const uint32_t xi = __reduce_add_sync(0xffffffffu, Lin);
    const uint32_t xo = __reduce_add_sync(0xffffffffu, D);
    if (lane == 0 && xi) atomicAdd(&s_cnt[6], (unsigned long long)xi);
    if (lane == 0 && xo) atomicAdd(&s_cnt[7], (unsigned long long)xo);
}

__global__ void __launch_bounds__(F_THREADS, 1)
k_in_fused_ring_pipe(DevTable T, InState S, const InBatchArgs *slots, RingRun R, uint32_t hmask,
                     InPipeBufs P)
{
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t n_slots = R.n_slots, n_batches = R.n_batches, first = R.first;
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x;
    if (n_batches == 0) return;
    if (!NBA_RING_TRACE && R.ts && cta == 0 && tid == 0) R.ts[0] = gtimer();
    const uint32_t base0 = *reinterpret_cast<volatile uint32_t *>(&S.ctl[CTLI_BASE]);
    // (no row-scan arrival of this launch precedes every CTA's first tile
    // arrival, which follows this read)
    const uint32_t base2 = *reinterpret_cast<volatile uint32_t *>(&S.ctl[CTLI_BAR2]);
    const uint32_t sb = smem_u32(smem);
    const uint32_t toff = (0x10000u - (sb & 0xffffu)) & 0xffffu;
    uint32_t lo_off = 0;
    if (toff < sizeof(FusedLo)) {
        if (toff + AES_TABLE_BYTES + sizeof(FusedHi) + sizeof(FusedLo) > F_SMEM) __trap();
        lo_off = toff + AES_TABLE_BYTES + (uint32_t)sizeof(FusedHi);
    }
    uint8_t *tabs = smem + toff;
    FusedLo &L = *reinterpret_cast<FusedLo *>(smem + lo_off);
    FusedHi &H = *reinterpret_cast<FusedHi *>(smem + toff + AES_TABLE_BYTES);
    const uint32_t lane4r = (lane * 4u) | (smem_u32(tabs) & 0xffff0000u);
    uint4 *scr = P.scr + (size_t)cta * PIPE_MAX_PPC;
    // the duplicate hash of batch k: H[k mod 4] (H0 = S.hkey / S.hval)
    auto hk_of = [&](uint32_t k) {
        const uint32_t m = k & 3u;
        return m == 0u ? S.hkey : m == 1u ? P.hk1 : m == 2u ? P.hk2 : P.hk3;
    };
    auto hv_of = [&](uint32_t k) {
        const uint32_t m = k & 3u;
        return m == 0u ? S.hval : m == 1u ? P.hv1 : m == 2u ? P.hv2 : P.hv3;
    };
    __shared__ unsigned long long s_cnt[N_IN_COUNTERS - 1];   // the CTA's decision counters
    if (tid < N_IN_COUNTERS - 1) s_cnt[tid] = 0ull;
    tables_stage(tabs, T, &L.tbar, true);   // bulk copy, waited for before the first lookup
    if (tid < NBINS) L.bins[tid] = 0u;
    // batches 0 and 1's duplicate hashes, cleared by every CTA before a start
    // barrier that the first inserts (after batch 0's lanes) follow
    for (uint32_t k = cta * F_THREADS + tid; k <= hmask; k += G * F_THREADS) {
        S.hkey[k] = ~0ull;
        S.hval[k] = ~0u;
        P.hk1[k] = ~0ull;
        P.hv1[k] = ~0u;
    }
    __syncthreads();
    grid_arrive(&S.ctl[CTLI_BAR]);
    const bool isP = tid >= PIPE_MAX_PPC;
    const uint32_t pt = tid - PIPE_MAX_PPC;
    auto ppc_of = [&](const InBatchArgs &B) {
        uint32_t ppc = (B.n + G - 1) / G;
        ppc = (ppc + 31u) & ~31u;
        return ppc < 32u ? 32u : ppc;
    };
    if (isP) {
        const InBatchArgs B0 = slots[first % n_slots];
        in_pipe_prologue(T, B0, ppc_of(B0), L, pt);
    }
    __syncthreads();
    tables_bulk_wait(&L.tbar, 0u);
    grid_wait(&S.ctl[CTLI_BAR], base0 + G);          // the start barrier (long since complete)
    // per CTA and batch k: its tile part arrives at CTLI_BAR (SB1(k) complete
    // at bbase + (k + 1) G) and its row scans at CTLI_BAR2 (SB2(k) at
    // base2 + (k + 1) G)
    const uint32_t bbase = base0 + G;
    for (uint32_t bi = 0; bi < n_batches; bi++) {
        const InBatchArgs B = slots[(first + bi) % n_slots];
        const uint32_t ppc = ppc_of(B);
        const uint32_t p_begin = cta * ppc;
        const uint32_t p_end = min(B.n, p_begin + ppc);
        const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
#if NBA_RING_TRACE
        unsigned long long *tr = IRTR(bi, 0);
        if (tr && tid == 0) tr[0] = gtimer();
#else
        unsigned long long *tr = nullptr;
#endif
        if (!isP) {
            unsigned long long *hk = hk_of(bi);
            uint32_t *hv = hv_of(bi);
            const uint32_t run = L.wrun[warp];
            const uint32_t pos = 32u * run + lane;
            const bool have = run != 0xffu && pos < cnt;
            const uint32_t pk = have ? L.perm[pos] : 0u;
            uint32_t info = have ? L.info[pk] : 0u;
            const uint32_t sa_raw = have ? L.sa[pk] : INVALID_SA;   // (the tail tells DROP_SA apart)
            uint32_t q = have ? L.seq[pk] : 0u;          // (NBA_IN_LANE_FORMAT: the outer length)
            uint32_t iv0 = have ? L.aux0[pk] : 0u, iv1 = have ? L.aux1[pk] : 0u;
            const uint32_t inoff = have ? L.inoff[pk] : 0u, outoff = have ? L.outoff[pk] : 0u;
            bar_arrive_n(2, F_THREADS);                  // fields taken: the arrays are free
            if (NBA_IN_LANE_ROWS && bi > 0)              // batch bi - 1's row scans, bi + 2's hash
                in_pipe_rows_lanes(T, S, hmask, bbase + bi * G, hk_of(bi + 2), hv_of(bi + 2), tr);
            if (NBA_IN_LANE_FORMAT && have) in_format(T, B, sa_raw, q, inoff, info, q, iv0, iv1);
            const uint32_t sa = (info & INFO_OK) ? sa_raw : INVALID_SA;
            if (have) {
                uint32_t flags = 0;
                if (info & INFO_OK) {
                    uint4 r0, hd, h0, h1, r1, r2;
                    const uint4 *line = T.sal + (size_t)sa * SAL_U4;
                    ldg_nc_v8(&line[0], r0, hd);
                    ldg_nc_v8(&line[2], h0, h1);
                    expand_key_lane(lane4r, r0, r1, r2, L, H, tid);
                    flags = INF_FMT | esp_in_packet(T, B, L, H, lane4r, tid, sa, info & 0xffffu, q, iv0,
                                                    iv1, inoff, outoff, r0, r1, r2, hd, h0, h1);
                    // (sa, q) -> first index into batch bi's duplicate hash
                    // (cleared during batch bi - 2, read by batch bi's
                    // decisions during batch bi + 1): the atomics' latency
                    // overlaps the other lanes' crypto
                    if (flags & INF_ICV) replay_hash_insert(hk, hv, sa, q, p_begin + pk, hmask);
                }
                L.tailf[pk] = flags;
                L.tailq[pk] = q;
                L.tails[pk] = sa_raw;
            }
            if (tr && lane == 0) atomicMax(&tr[3], gtimer());
            if (bi > 0) {
                // batch bi - 1's decisions for this warp's 32 packet slots,
                // once every CTA's side warps scanned their rows (SB2)
                const InBatchArgs Bp = slots[(first + bi - 1) % n_slots];
                in_pipe_decide(T, S, Bp, ppc_of(Bp), scr, hmask, hk_of(bi - 1), hv_of(bi - 1),
                               base2 + bi * G, warp, s_cnt);
                if (tr && lane == 0) atomicMax(&tr[9], gtimer());
            }
        } else {
            bar_sync_n(2, F_THREADS);                    // every lane took its fields
            // batch bi - 1's row scans and batch bi + 2's hash cleared (its
            // last user, batch bi - 2, decided before every CTA's tile part
            // of batch bi - 1), and batch bi + 1's prologue
            const bool more = bi + 1 < n_batches;
            if (NBA_IN_PREFETCH && more) {
                const InBatchArgs Bn = slots[(first + bi + 1) % n_slots];
                in_pipe_prefetch_hdr(Bn, ppc_of(Bn), pt);
                if (bi + 2 < n_batches) {
                    const InBatchArgs Bm = slots[(first + bi + 2) % n_slots];
                    in_pipe_prefetch_meta(Bm, ppc_of(Bm), pt);
                }
            }
            if (NBA_IN_PRO_FIRST && more) {
                const InBatchArgs Bn = slots[(first + bi + 1) % n_slots];
                in_pipe_prologue(T, Bn, ppc_of(Bn), L, pt, tr);
            }
            if (bi > 0) {
                if (!NBA_IN_LANE_ROWS)
                    in_pipe_rows(T, S, hmask, bbase + bi * G, hk_of(bi + 2), hv_of(bi + 2), pt, tr);
            } else {
                for (uint32_t k = cta * PIPE_P + pt; k <= hmask; k += G * PIPE_P) {
                    P.hk2[k] = ~0ull;
                    P.hv2[k] = ~0u;
                }
            }
            if (!NBA_IN_PRO_FIRST && more) {
                const InBatchArgs Bn = slots[(first + bi + 1) % n_slots];
                in_pipe_prologue(T, Bn, ppc_of(Bn), L, pt, tr);
            }
            if (tr && pt == 0) tr[4] = gtimer();
        }
        if (bi > 0 && tid == 0) {
            // every CTA (also one without packets in batch bi - 1, whose lanes
            // did not wait) passes SB2(bi - 1) before its tile part rewrites
            // the tile maxima that batch bi - 1's row scans read
            uint32_t v;
            do {
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&S.ctl[CTLI_BAR2]) : "memory");
            } while ((int)(v - (base2 + bi * G)) < 0);
        }
        __syncthreads();                                  // lanes done, bi - 1 decided, bi + 1 prepared
        if (!NBA_RING_TRACE && R.ts && bi > 0 && tid == 0) atomicMax(&R.ts[bi], gtimer());
        in_pipe_tile(S, L, H, cnt, scr);                  // (ends with the SB1(bi) arrival)
        if (tr && tid == 0) tr[6] = gtimer();
        __syncthreads();                                  // the tile part's scratch is free again
#if NBA_RING_TRACE
        if (tr && tid == 0) tr[5] = gtimer();
#endif
    }
    // the last batch's replay: row scans by the side warps, decisions by the lane warps
    const uint32_t bl = n_batches - 1u;
    if (isP) {
        if (!NBA_IN_LANE_ROWS) in_pipe_rows(T, S, hmask, bbase + (bl + 1u) * G, nullptr, nullptr, pt, nullptr);
    } else {
        if (NBA_IN_LANE_ROWS) in_pipe_rows_lanes(T, S, hmask, bbase + (bl + 1u) * G, nullptr, nullptr, nullptr);
        const InBatchArgs Bp = slots[(first + bl) % n_slots];
        in_pipe_decide(T, S, Bp, ppc_of(Bp), scr, hmask, hk_of(bl), hv_of(bl), base2 + (bl + 1u) * G, warp,
                       s_cnt);
    }
    __syncthreads();
    if (tid < N_IN_COUNTERS - 1 && s_cnt[tid]) atomicAdd(&S.counters[tid], s_cnt[tid]);
    if (!NBA_RING_TRACE && R.ts && tid == 0) atomicMax(&R.ts[1u + bl], gtimer());
    if (tid == 0 && cta == 0) {
        atomicAdd(&S.counters[N_IN_COUNTERS - 1], (unsigned long long)n_batches);
        S.ctl[CTLI_BASE] = bbase + n_batches * G;        // a start barrier, one tile arrival per batch
    }
}

cudaError_t launch_in_fused_ring_pipe(const DevTable &T, const InState &S, const InBatchArgs *slots,
                                      const RingRun &R, uint32_t hmask, const InPipeBufs &P, int grid,
                                      cudaStream_t st)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(F_THREADS);
    cfg.dynamicSmemBytes = F_SMEM;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;   // grid barriers inside
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_in_fused_ring_pipe, T, S, slots, R, hmask, P);
}

bool in_pipe_ok(uint32_t n, int grid)
{
    uint32_t ppc = (n + grid - 1) / grid;
    ppc = (ppc + 31u) & ~31u;
    return n > 0 && grid <= 160 && ppc <= PIPE_MAX_PPC;
}

cudaError_t launch_in_fused_ring(const DevTable &T, const InState &S, const InBatchArgs *slots,
                                 const RingRun &R, uint32_t hmask,
                                 unsigned long long *hkey_b, uint32_t *hval_b, int grid,
                                 cudaStream_t st)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(F_THREADS);
    cfg.dynamicSmemBytes = F_SMEM;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;   // grid barriers inside
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_in_fused_ring, T, S, slots, R, hmask, hkey_b, hval_b);
}

cudaError_t launch_in_fused(const DevTable &T, const InState &S, const InHashPair &HP,
                            const InBatchArgs &B, int grid, uint32_t hmask, uint32_t hfull,
                            bool merged, uint32_t *bar_base, cudaStream_t st)
{
    uint32_t ppc = (B.n + grid - 1) / grid;
    ppc = (ppc + 31u) & ~31u;
    if (ppc < 32u) ppc = 32u;
    const uint32_t g = (B.n + ppc - 1) / ppc;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(g);
    cfg.blockDim = dim3(F_THREADS);
    cfg.dynamicSmemBytes = F_SMEM;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;   // grid barriers inside (merged)
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = merged ? 1 : 0;
    (void)bar_base;   // the one-kernel form keeps its barrier base on the device
    cudaError_t e = merged ? cudaLaunchKernelEx(&cfg, k_in_fused<true>, T, S, HP, B, ppc, hmask, hfull, 0u)
                           : cudaLaunchKernelEx(&cfg, k_in_fused<false>, T, S, HP, B, ppc, hmask, hfull, 0u);
    return e;
}

bool in_merged_ok(uint32_t n, int grid)
{
    uint32_t ppc = (n + grid - 1) / grid;
    ppc = (ppc + 31u) & ~31u;
    return ppc <= (uint32_t)F_SUPER;
}

cudaError_t setup_in_fused_attributes()
{
    cudaError_t e = cudaFuncSetAttribute(k_in_fused_ring, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)F_SMEM);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(k_in_fused_ring_pipe, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)F_SMEM);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(k_in_fused<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)F_SMEM);
    if (e != cudaSuccess) return e;
    return cudaFuncSetAttribute(k_in_fused<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)F_SMEM);
}

}  // namespace nba
