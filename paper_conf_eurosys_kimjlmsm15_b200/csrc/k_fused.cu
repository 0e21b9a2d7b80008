// k_fused.cu -- rows a2..a5 in ONE persistent kernel (the
// datablock-reuse / copy-coalescing optimisation NBA left as future work,
// PAPER.md:329 and :345).
//
// One 512-thread CTA per SM shares one 128 KB bank-replicated T-table image.
// Each CTA owns a contiguous packet range and walks it in super-rounds of up to
// F_SUPER packets:
//   1. all threads, one packet each: validity, sizes, ESP sequence number (from
//      the prologue's per-SA ranks), and a CTA-local counting sort by SHA-1
//      length (longest first) so the 32 lanes of a warp get equal work;
//   2. one LANE per packet, in 64-byte steps: read 64 payload bytes straight
//      from the caller's buffer (pad / trailer appended), encrypt the 4 RFC 3686
//      counter blocks with the table AES (rounds 1-2 from a per-packet CTR
//      precompute), stream the ciphertext to its final place in the output slot
//      with destination-aligned 16-byte stores, and immediately compress the
//      SHA-1 block that this ciphertext completes (HMAC-SHA1-96 from the SA's
//      precomputed midstates); finally the outer hash and the ICV.
// Within a lane, AES (shared-memory LSU bound) and SHA-1 (ALU bound) alternate
// every 64 bytes, so across the SM's warps both pipes are busy at once; every
// payload byte is read from HBM once and written once, and no data or
// synchronisation crosses lanes.
//
// Shared-memory layout: the T-tables sit at a 64 KB-aligned shared-window
// address, so a single PRMT forms the complete LDS address of a lookup
// (byte r of the state word in bits 8..15, lane*4 in bits 0..7, the table base
// in bits 16..31) -- no address add per lookup.  Per-thread round keys and the
// packet metadata live below (FusedLo) and above (FusedHi) the tables.
#include <cstdlib>

#include "fused_common.cuh"

namespace nba {

#ifndef NBA_PF_AHEAD          // payload prefetch distance in 64-byte steps
#define NBA_PF_AHEAD 3
#endif
#ifndef NBA_LONG_HIGH         // 1: longest packets in the highest warps (A/B: lowest is faster)
#define NBA_LONG_HIGH 0
#endif
#ifndef NBA_INTERIOR          // 1: select-free fast path for interior 64-byte steps / SHA blocks
#define NBA_INTERIOR 1
#endif
#ifndef NBA_EXPAND_MID        // merged: expand round keys after the row scans (1) or before the barrier wait (0)
#define NBA_EXPAND_MID 0
#endif
#ifndef NBA_POLL_NS           // back-off between polls of a sequence-number base (ns)
#define NBA_POLL_NS 0
#endif
#ifndef NBA_LDG256            // 1: payload steps as three 256-bit loads (else five 128-bit)
#define NBA_LDG256 1
#endif
#ifndef NBA_CARRY             // 1: reuse the previous step's last 32-byte payload block
#define NBA_CARRY 0
#endif
#ifndef NBA_HDR_DEFER         // 1: the outer header words go out with the first ciphertext words
#define NBA_HDR_DEFER 0       //   (one put16 of header + 7 ciphertext words, its SA-line words and TOS
#endif                        //   byte re-read; esp_packet<true>): measured per kernel
#ifndef NBA_STG256            // 1: output through 32-byte chunks (256-bit stores)
#define NBA_STG256 0
#endif
#ifndef NBA_RK_ASYNC          // pipelined ring: round keys 3..10 by cp.async from the SA's
#define NBA_RK_ASYNC 0        //   schedule (1) instead of expanded in the lane (0); measured
#endif                        //   slower (64 B 24.4 -> 27.5 us: the LDGSTS issue delays the scans)
#ifndef NBA_PIPE_STAGGER      // pipelined ring: lane warps 7..13 start their packets later by
#define NBA_PIPE_STAGGER 128  //   STAGGER/256 x the time the lower warps took to their first AES
#endif                        //   step (previous batch), so AES (LDS) and SHA-1 (ALU) overlap
#ifndef NBA_PIPE_SPLIT        // pipelined ring: batches of one-AES-step packets run on producer
#define NBA_PIPE_SPLIT 0      //   (AES) and consumer (SHA-1) warps (split_produce / _consume);
#endif                        //   measured slower (64 B 23.7 -> 27.4 us), off
#ifndef NBA_PIPE_PRO_DELAY    // pipelined ring: the prologue warps start the next batch's work
#define NBA_PIPE_PRO_DELAY 1  //   min(4 us, 1/4 of the previous batch's lane phase) after the
#endif                        //   lanes took their fields (off the AES phase's shared-memory load)
#ifndef NBA_PIPE_ONEBIN       // pipelined ring: one-length-bin batches keep index order (no sort)
#define NBA_PIPE_ONEBIN 1
#endif
#ifndef NBA_PIPE_PRO_DELAY0   // the prologue warps' delay in the first iteration of a launch (ns)
#define NBA_PIPE_PRO_DELAY0 0
#endif
#ifndef NBA_PIPE_META_PF      // pipelined ring: L2 prefetch of the metadata two batches ahead
#define NBA_PIPE_META_PF 1
#endif
#ifndef NBA_SA_PREFETCH       // L2 prefetch of the SA table at kernel start
#define NBA_SA_PREFETCH 1
#endif


// ---------------------------------------------- one packet, one lane
// The packet's SA-table words (round keys 0..2, header words, inner HMAC
// midstate) and the inner TOS byte: loaded together so their latencies
// overlap; the merged kernel issues them before it waits at its grid barrier.
struct PktPre {
    uint4 r0, r1, r2, hd, h0, h1;
    uint32_t tos;
};

// Loads the SA line (one 128-byte line per SA) and the TOS byte; r1 / r2 are
// filled in by expand_key_lane.
__device__ __forceinline__ PktPre load_pkt_pre(const DevTable &T, const uint8_t *in_buf, uint32_t sa,
                                               uint32_t inoff, bool load_tos, uint32_t tos)
{
    PktPre p;
    const uint4 *line = T.sal + (size_t)sa * SAL_U4;
    ldg_nc_v8(&line[0], p.r0, p.hd);
    ldg_nc_v8(&line[2], p.h0, p.h1);
    p.r1 = p.r2 = make_uint4(0, 0, 0, 0);
    // TOS of the inner header (the outer header copies it, reading A13)
    p.tos = load_tos ? (uint32_t)__ldg(in_buf + inoff + 1) : tos;
    return p;
}

template <bool HDR_DEFER = (NBA_HDR_DEFER != 0)>
__device__ __forceinline__ void esp_packet(const DevTable &T, const BatchArgs &B, FusedLo &L,
                                           FusedHi &H, uint32_t lane4r, uint32_t tid, uint32_t sa,
                                           uint32_t info, uint32_t q32, uint32_t inoff,
                                           uint32_t outoff, const PktPre &pp, unsigned long long *dbg,
                                           uint32_t *aes0_mark = nullptr, uint32_t t_start = 0,
                                           uint32_t skip = 0)
{
    // skip (the role-split lanes' warm-up pass only; 0 for every real packet):
    // bit 0 the CTR precompute, 1 the AES step and its emission, 3 the SHA-1
    // compressions -- warps entering the code at different points fetch its
    // instruction lines in parallel
    long long ck_start = clock64(), ck_setup = 0, ck_aes = 0, ck_sha = 0, ck_emit = 0;
    const uint4 r0 = pp.r0, r1 = pp.r1, r2 = pp.r2, hd = pp.hd, h0 = pp.h0, h1 = pp.h1;
    const uint32_t D = info & 0x7ffu;
    const uint32_t tos = pp.tos;
    const uint32_t pad = esp_pad(D);
    const uint32_t C = D + pad + 2u;
    const uint32_t Lb = 48u + C;
    const uint32_t Cw = C >> 2;                  // ciphertext words
    const uint32_t Mw = 4u + Cw;                 // MAC input words (ESP hdr + ciphertext)
    const uint32_t nsteps = (Cw + 15u) >> 4;     // 64-byte AES steps
    const uint32_t nb_in = (4u * Mw + 8u) / 64u + 1u;   // inner SHA-1 blocks
    const uint32_t bitlen = (64u + 4u * Mw) * 8u;        // the ipad block counts

    // ---- per-packet setup: round keys, CTR precompute (FIPS-197 rounds 1-2 on
    // nonce || 0 || BE32(q) || BE32(k+1), k+1 < 256: only byte 3 of column 3
    // varies, so round 1 is t0 = T3[r3 ^ (k+1)] ^ X0 and round 2 is
    // u_c = T[row(t0)] ^ Z_c), header words, HMAC inner midstate
    // round keys 3..10 were expanded into L.rkA / H.rkB[.][tid] by expand_key_lane
    const uint32_t qbe = bswap32(q32);
    CtrPre cp{};
    if (!(skip & 1u)) cp = ctr_precompute(lane4r, r0, r1, r2, hd.y, 0u, qbe);   // IV = BE64(q), A6

    // outer IPv4 header (reading A13) + ESP header + IV: output words 0..8
#if NBA_STG256
    OutStream32 os;
#else
    OutStream os;
#endif
    os.init(B.out_buf + outoff);
    // outer header words 0..8; emitted together with the first ciphertext words
    // (NBA_HDR_DEFER: one 16-word put16 instead of 16 single-word puts for
    // packets of >= 7 ciphertext words), else right here
    auto header_words = [&](uint32_t (&h)[9]) {
        const uint32_t src = bswap32(hd.z), dst = bswap32(hd.w);
        uint32_t sum = (0x4500u | tos) + Lb + 0x4000u + ((64u << 8) | 50u) + (src >> 16) +
                       (src & 0xffffu) + (dst >> 16) + (dst & 0xffffu);
        sum = (sum & 0xffffu) + (sum >> 16);
        sum = (sum & 0xffffu) + (sum >> 16);
        const uint32_t cs = ~sum & 0xffffu;
        h[0] = 0x45u | (tos << 8) | ((Lb >> 8) << 16) | ((Lb & 0xffu) << 24);
        h[1] = 0x00400000u;
        h[2] = 64u | (50u << 8) | ((cs >> 8) << 16) | ((cs & 0xffu) << 24);
        h[3] = hd.z;
        h[4] = hd.w;
        h[5] = hd.x;
        h[6] = qbe;
        h[7] = 0u;
        h[8] = qbe;
    };
    // (NBA_HDR_RELOAD: the deferred header re-reads its SA-line words and the
    // inner TOS byte instead of keeping them live across the AES step)
    auto header_words_reload = [&](uint32_t (&h)[9]) {
        const uint4 hd2 = ldg_nc_v4(&T.sal[(size_t)sa * SAL_U4 + 1]);
        const uint32_t tos2 = (uint32_t)__ldg(B.in_buf + inoff + 1);
        const uint32_t src = bswap32(hd2.z), dst = bswap32(hd2.w);
        uint32_t sum = (0x4500u | tos2) + Lb + 0x4000u + ((64u << 8) | 50u) + (src >> 16) +
                       (src & 0xffffu) + (dst >> 16) + (dst & 0xffffu);
        sum = (sum & 0xffffu) + (sum >> 16);
        sum = (sum & 0xffffu) + (sum >> 16);
        const uint32_t cs = ~sum & 0xffffu;
        h[0] = 0x45u | (tos2 << 8) | ((Lb >> 8) << 16) | ((Lb & 0xffu) << 24);
        h[1] = 0x00400000u;
        h[2] = 64u | (50u << 8) | ((cs >> 8) << 16) | ((cs & 0xffu) << 24);
        h[3] = hd2.z;
        h[4] = hd2.w;
        h[5] = hd2.x;
        h[6] = qbe;
        h[7] = 0u;
        h[8] = qbe;
    };
    const bool hdr_defer = HDR_DEFER && Cw >= 7u;
    if (!hdr_defer) {
        uint32_t h[9];
        header_words(h);
#pragma unroll
        for (int w = 0; w < 9; w++) os.put(h[w]);
    }
    // SHA-1 message words 0..3 = ESP header (big-endian words of the wire bytes)
    uint32_t carry[4] = {bswap32(hd.x), q32, 0u, q32};
    uint32_t st[5] = {h0.x, h0.y, h0.z, h0.w, h1.x};
    const uint8_t *src = B.in_buf + inoff;
    const uintptr_t src_end = reinterpret_cast<uintptr_t>(src) + D;
    ck_setup = clock64();
    // payload steps 1 and 2 into L2 ahead of use (step 0 was touched by the
    // metadata phase); each step prefetches two steps ahead
#pragma unroll
    for (uint32_t k = 1; k < NBA_PF_AHEAD; k++)
        if (D > 64u * k) prefetch_bytes(src + 64u * k, min(64u, D - 64u * k));

    // ---- one SHA-1 compression per iteration; AES steps feed the first nsteps
#pragma unroll 1
    uint4 pcarry0 = make_uint4(0, 0, 0, 0), pcarry1 = pcarry0;   // NBA_CARRY: last payload block
    for (uint32_t it = 0; it <= nb_in; it++) {
        uint32_t ct[16];
#pragma unroll
        for (int w = 0; w < 16; w++) ct[w] = 0u;
        if (it < nsteps && !(skip & 2u)) {
            // payload words of T bytes [64 it, 64 it + 64), realigned
            if (64u * (it + NBA_PF_AHEAD) < D)
                prefetch_bytes(src + 64u * (it + NBA_PF_AHEAD), min(64u, D - 64u * (it + NBA_PF_AHEAD)));
            // interior step: all 16 words are payload, the trailer (last word and,
            // when p = 3, the one before) lies beyond it, and the five 16-byte
            // loads are inside the datagram -- no per-word selects, one bounds test
            const bool interior = NBA_INTERIOR && 16u * it + 18u <= Cw;
#if NBA_LDG256 && NBA_CARRY
            // block 0 of this step is block 2 of the previous one (the stream
            // advances 64 bytes = two 32-byte blocks per step): two new loads
            Raw6 raw;
            {
                const uintptr_t a = reinterpret_cast<uintptr_t>(src) + 64u * it;
                const uintptr_t abase = a & ~(uintptr_t)31;
                raw.sh = (uint32_t)(a & 31u);
                if (it == 0) {
                    if (abase < src_end) ldg_nc_v8(reinterpret_cast<const void *>(abase), raw.c[0], raw.c[1]);
                    else raw.c[0] = raw.c[1] = make_uint4(0, 0, 0, 0);
                } else {
                    raw.c[0] = pcarry0;
                    raw.c[1] = pcarry1;
                }
#pragma unroll
                for (int i = 1; i < 3; i++) {
                    const uintptr_t qa = abase + 32u * i;
                    if (interior || qa < src_end) ldg_nc_v8(reinterpret_cast<const void *>(qa), raw.c[2 * i], raw.c[2 * i + 1]);
                    else raw.c[2 * i] = raw.c[2 * i + 1] = make_uint4(0, 0, 0, 0);
                }
                pcarry0 = raw.c[4];
                pcarry1 = raw.c[5];
            }
#elif NBA_LDG256
            Raw6 raw;
            if (interior) load_raw6_inb(reinterpret_cast<uintptr_t>(src) + 64u * it, raw);
            else load_raw6(reinterpret_cast<uintptr_t>(src) + 64u * it, src_end, raw);
#else
            Raw5 raw;
            if (interior) load_raw5_inb(reinterpret_cast<uintptr_t>(src) + 64u * it, raw);
            else load_raw5(reinterpret_cast<uintptr_t>(src) + 64u * it, src_end, raw);
#endif
            // AES-128 of counter blocks 4 it + 1 .. 4 it + 4
            uint32_t ks[16];
            aes4_keystream(lane4r, cp, it, L, H, tid, ks);
            // plaintext T = P || pad || p || 4, XOR keystream
            {
                extract16(raw, ct);
                // trailer: T ends on a word boundary (C = 0 mod 4), so it touches only
                // the last word (and the one before when p = 3):
                //   p=0 [P P 0 4]  p=1 [P 1 1 4]  p=2 [1 2 2 4]  p=3 [.. 1][2 3 3 4]
                if (!interior) {
                    const uint32_t lw = Cw - 1u - 16u * it;          // last T word in this step?
                    const uint32_t keep = pad == 0 ? 0x0000ffffu : pad == 1 ? 0x000000ffu : 0u;
                    const uint32_t trl = pad == 0 ? 0x04000000u : pad == 1 ? 0x04010100u
                                       : pad == 2 ? 0x04020201u : 0x04030302u;
#pragma unroll
                    for (int w = 0; w < 16; w++) {
                        if ((uint32_t)w == lw) ct[w] = (ct[w] & keep) | trl;
                        if (pad == 3u && (uint32_t)w + 1u == lw) ct[w] = (ct[w] & 0x00ffffffu) | 0x01000000u;
                    }
                    if (pad == 3u && lw == 16u) ct[15] = (ct[15] & 0x00ffffffu) | 0x01000000u;
                }
#pragma unroll
                for (int w = 0; w < 16; w++) ct[w] ^= ks[w];
            }
            long long ck_a1 = clock64();
            ck_aes += 0;
            // pipelined ring: how long the lower lane warps take to their first
            // AES step (the upper ones start that much later next batch)
            if (aes0_mark && it == 0) atomicMax(aes0_mark, (uint32_t)gtimer() - t_start);
            // stream the ciphertext words of this step to the output slot
            if (hdr_defer && it == 0u) {
                uint32_t v[16];
                uint32_t h[9];
                header_words_reload(h);
#pragma unroll
                for (int w = 0; w < 9; w++) v[w] = h[w];
#pragma unroll
                for (int w = 0; w < 7; w++) v[9 + w] = ct[w];
                os.put16(v);
#pragma unroll
                for (int w = 7; w < 16; w++)
                    if ((uint32_t)w < Cw) os.put(ct[w]);
            } else if (16u * it + 16u <= Cw) {
                os.put16(ct);
            } else {
#pragma unroll
                for (int w = 0; w < 16; w++)
                    if (16u * it + w < Cw) os.put(ct[w]);
            }
            if (it == 0) { ck_aes = ck_a1; ck_emit = clock64(); }
        }
        // SHA-1 block: inner block `it` (message words 16 it .. 16 it + 15 with
        // FIPS 180-4 §5.1.1 padding), or the outer hash of the inner digest
        uint32_t W[16];
        if (it < nb_in) {
            const uint32_t m0 = 16u * it;
            if (NBA_INTERIOR && m0 + 16u <= Mw && it + 1u < nb_in) {   // a block of message words only
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
        if (!(skip & 8u)) sha1_compress_fma(st, W, T.n_sa != 0u ? 1u : 0u);   // (n_sa >= 1: an opaque 1)
        if (it == 0) ck_sha = clock64();
    }
    // ICV = first 96 bits of the outer digest (RFC 2404)
    os.put(bswap32(st[0]));
    os.put(bswap32(st[1]));
    os.put(bswap32(st[2]));
    os.finish(B.out_buf + outoff + Lb);
    if (dbg) {
        long long ck_end = clock64();
        dbg[0] = ck_setup - ck_start;      // setup (round keys, precompute, header)
        dbg[1] = ck_aes - ck_setup;        // payload + AES step 0 (+ pt build)
        dbg[2] = ck_emit - ck_aes;         // ciphertext emission step 0
        dbg[3] = ck_sha - ck_emit;         // SHA block 0
        dbg[4] = ck_end - ck_sha;          // the rest
        dbg[5] = st[0];
    }
}

// ---------------------------------- one-step packets, producer / consumer warps
// For a batch whose packets all fit one 64-byte AES step (C <= 64: frames up to
// 76 bytes), the pipelined ring can split each packet's work between two
// kinds of warps instead of one lane doing AES then SHA-1: PRODUCER threads
// (warps 0..5) run the AES-CTR step and write the ciphertext into a shared
// staging slot, CONSUMER threads (warps 6..13) wait for it and run the three
// SHA-1 compressions and the output stream.  With every lane doing AES first
// and SHA-1 second, the SM's shared-memory pipe and ALU pipe take turns;
// split, the shared-memory-bound AES of some packets runs beside the ALU-bound
// SHA-1 of others.  Same arithmetic and results as esp_packet.
constexpr uint32_t SPLIT_PROD = 192;          // producer threads (warps 0..5)
constexpr uint32_t SPLIT_CONS = PIPE_MAX_PPC - SPLIT_PROD;          // 256 consumers

// Producer: packet with datagram length D, sequence number q32: the 16 words
// of T xor keystream (C <= 64) into the staging slot ct[0..3][j] (uint4 x 4).
__device__ __forceinline__ void split_produce(const DevTable &T, const BatchArgs &B, FusedLo &L,
                                              FusedHi &H, uint32_t lane4r, uint32_t slot, uint32_t sa,
                                              uint32_t info, uint32_t q32, uint32_t inoff, uint32_t j)
{
    const uint32_t D = info & 0x7ffu;
    const uint32_t pad = esp_pad(D);
    const uint32_t C = D + pad + 2u;
    const uint32_t Cw = C >> 2;
    uint4 r0, hd, r1, r2;
    const uint4 *line = T.sal + (size_t)sa * SAL_U4;
    ldg_nc_v8(&line[0], r0, hd);
    const uint8_t *src = B.in_buf + inoff;
    // round keys 3..6 -> L.rkA[.][slot], 7..10 -> L.rkA[.][256 + slot]
    uint4 *rkl = &L.rkA[0][0], *rkh = &L.rkA[0][256];
    expand_key_slots(lane4r, r0, r1, r2, rkl, rkh, slot);
    const CtrPre cp = ctr_precompute(lane4r, r0, r1, r2, hd.y, 0u, bswap32(q32));
    Raw6 raw;      // the payload's loads in flight during the AES rounds
    load_raw6(reinterpret_cast<uintptr_t>(src), reinterpret_cast<uintptr_t>(src) + D, raw);
    uint32_t ks[16], ct[16];
    aes4_keystream(lane4r, cp, 0u, rkl, rkh, slot, ks);
    extract16(raw, ct);
    {   // trailer (C = 0 mod 4): the last word and, when p = 3, the one before
        const uint32_t lw = Cw - 1u;
        const uint32_t keep = pad == 0 ? 0x0000ffffu : pad == 1 ? 0x000000ffu : 0u;
        const uint32_t trl = pad == 0 ? 0x04000000u : pad == 1 ? 0x04010100u
                           : pad == 2 ? 0x04020201u : 0x04030302u;
#pragma unroll
        for (int w = 0; w < 16; w++) {
            if ((uint32_t)w == lw) ct[w] = (ct[w] & keep) | trl;
            if (pad == 3u && (uint32_t)w + 1u == lw) ct[w] = (ct[w] & 0x00ffffffu) | 0x01000000u;
        }
    }
#pragma unroll
    for (int w = 0; w < 16; w++) ct[w] ^= ks[w];
    uint4 *stg = &H.rkB[0][0];
#pragma unroll
    for (int k = 0; k < 4; k++)
        stg[k * F_THREADS + j] = make_uint4(ct[4 * k], ct[4 * k + 1], ct[4 * k + 2], ct[4 * k + 3]);
}

// Consumer: the staged ciphertext of packet j -> outer header, ESP header,
// ciphertext, HMAC-SHA1-96 (as esp_packet's SHA-1 part, one AES step).
__device__ __forceinline__ void split_consume(const DevTable &T, const BatchArgs &B, FusedHi &H,
                                              uint32_t sa, uint32_t info, uint32_t q32, uint32_t inoff,
                                              uint32_t outoff, uint32_t j)
{
    const uint32_t D = info & 0x7ffu;
    const uint32_t pad = esp_pad(D);
    const uint32_t C = D + pad + 2u;
    const uint32_t Lb = 48u + C;
    const uint32_t Cw = C >> 2;
    const uint32_t Mw = 4u + Cw;
    const uint32_t nb_in = (4u * Mw + 8u) / 64u + 1u;
    const uint32_t bitlen = (64u + 4u * Mw) * 8u;
    uint4 hd, h0, h1, dummy;
    const uint4 *line = T.sal + (size_t)sa * SAL_U4;
    ldg_nc_v8(&line[0], dummy, hd);
    ldg_nc_v8(&line[2], h0, h1);
    const uint32_t tos = (uint32_t)__ldg(B.in_buf + inoff + 1);
    const uint32_t qbe = bswap32(q32);
    uint32_t ct[16];
    {
        const uint4 *stg = &H.rkB[0][0];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint4 v = stg[k * F_THREADS + j];
            ct[4 * k] = v.x;
            ct[4 * k + 1] = v.y;
            ct[4 * k + 2] = v.z;
            ct[4 * k + 3] = v.w;
        }
    }
    OutStream os;
    os.init(B.out_buf + outoff);
    {
        const uint32_t src = bswap32(hd.z), dst = bswap32(hd.w);
        uint32_t sum = (0x4500u | tos) + Lb + 0x4000u + ((64u << 8) | 50u) + (src >> 16) +
                       (src & 0xffffu) + (dst >> 16) + (dst & 0xffffu);
        sum = (sum & 0xffffu) + (sum >> 16);
        sum = (sum & 0xffffu) + (sum >> 16);
        const uint32_t cs = ~sum & 0xffffu;
        os.put(0x45u | (tos << 8) | ((Lb >> 8) << 16) | ((Lb & 0xffu) << 24));
        os.put(0x00400000u);
        os.put(64u | (50u << 8) | ((cs >> 8) << 16) | ((cs & 0xffu) << 24));
        os.put(hd.z);
        os.put(hd.w);
        os.put(hd.x);
        os.put(qbe);
        os.put(0u);
        os.put(qbe);
    }
    if (Cw == 16u) {
        os.put16(ct);
    } else {
#pragma unroll
        for (int w = 0; w < 16; w++)
            if ((uint32_t)w < Cw) os.put(ct[w]);
    }
    uint32_t carry[4] = {bswap32(hd.x), q32, 0u, q32};
    uint32_t st[5] = {h0.x, h0.y, h0.z, h0.w, h1.x};
#pragma unroll 1
    for (uint32_t it = 0; it <= nb_in; it++) {
        uint32_t W[16];
        if (it < nb_in) {
            const uint32_t m0 = 16u * it;
#pragma unroll
            for (int i = 0; i < 16; i++) {
                const uint32_t m = m0 + i;
                const uint32_t msg = i < 4 ? carry[i] : (it == 0 ? bswap32(ct[i - 4]) : 0u);
                W[i] = m < Mw ? msg : (m == Mw ? 0x80000000u : 0u);
            }
            if (it == nb_in - 1u) W[15] = bitlen;
#pragma unroll
            for (int i = 0; i < 4; i++) carry[i] = bswap32(ct[12 + i]);
        } else {
#pragma unroll
            for (int i = 0; i < 5; i++) W[i] = st[i];
            W[5] = 0x80000000u;
#pragma unroll
            for (int i = 6; i < 15; i++) W[i] = 0u;
            W[15] = (64u + 20u) * 8u;
            uint4 g4, g5;
            ldg_nc_v8(&T.sal[(size_t)sa * SAL_U4 + 4], g4, g5);
            st[0] = g5.x; st[1] = g5.y; st[2] = g5.z; st[3] = g4.x; st[4] = g4.y;
        }
        sha1_compress_fma(st, W, T.n_sa != 0u ? 1u : 0u);
    }
    os.put(bswap32(st[0]));
    os.put(bswap32(st[1]));
    os.put(bswap32(st[2]));
    os.finish(B.out_buf + outoff + Lb);
}

// ------------------------------------------- merged prologue (row a1 in-kernel)
// When the whole batch fits in one super-round per CTA (n <= grid * F_SUPER),
// the prologue runs inside this kernel: each CTA is one tile.  Per-SA ranks in
// the CTA come from __match_any_sync groups merged across the 16 warps through
// a small shared hash (slot per SA; per-warp group sizes); the CTA's per-SA
// counts go to the SA-major matrix; after a grid barrier one warp per SA scans
// its row (exclusive prefix over CTAs, SA counter advance) and publishes
// epoch-tagged bases, which each packet polls.  Deterministic: no atomic
// decides a rank.  This part returns the packet's rank among the CTA's packets
// of its SA (INVALID_SA: not counted).
__device__ __forceinline__ uint32_t merged_local_rank(const DevWork &W, FusedLo &L, uint32_t s)
{
    constexpr uint32_t HS = 2u * F_SUPER, NW = F_THREADS / 32u;
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x;
    uint16_t(*wcnt)[NW] = reinterpret_cast<uint16_t(*)[NW]>(&L.rkA[0][0]);   // [HS][NW], 32 KB
    static_assert(sizeof(L.rkA) >= HS * NW * sizeof(uint16_t), "wcnt overlay");

    const uint32_t peers = __match_any_sync(0xffffffffu, s);
    const uint32_t leader = __ffs(peers) - 1, hi_lane = 31u - __clz(peers);
    const uint32_t wrank = __popc(peers & lanemask_lt()), wcnt_me = __popc(peers);
    uint32_t slot = 0;
    if (s != INVALID_SA && lane == leader) {
        slot = (s * 0x9E3779B1u) >> 22;                    // 10 bits -> HS = 1024
        while (true) {
            const uint32_t old = atomicCAS(&L.hkey[slot], INVALID_SA, s);
            if (old == INVALID_SA || old == s) break;
            slot = (slot + 1u) & (HS - 1u);
        }
        wcnt[slot][warp] = (uint16_t)wcnt_me;
        atomicOr(&L.hmask[slot], 1u << warp);
    }
    slot = __shfl_sync(0xffffffffu, slot, leader);
    __syncthreads();
    uint32_t rank = 0;
    if (s != INVALID_SA) {
        const uint32_t m = L.hmask[slot];
        uint32_t base = 0;
#pragma unroll
        for (uint32_t w = 0; w < NW; w++)
            if (w < warp && ((m >> w) & 1u)) base += wcnt[slot][w];
        rank = base + wrank;
        // the SA's last group in the CTA writes the CTA's count (nonzero only;
        // the row scan re-zeroes it)
        if ((m >> (warp + 1u)) == 0u && lane == hi_lane)
            W.hist16[(size_t)s * G + cta] = (uint16_t)(base + wcnt_me);
    }
    return rank;
}

// ---------------------------------------------------------------- the kernel
__host__ __device__ __forceinline__ uint32_t fused_ppc_hd(uint32_t n, uint32_t grid)
{
    uint32_t ppc = (n + grid - 1) / grid;
    ppc = (ppc + 31u) & ~31u;
    return ppc < 32u ? 32u : ppc;
}
#define fused_ppc(n, g) fused_ppc_hd((uint32_t)(n), (uint32_t)(g))

// One batch through the kernel (the body of k_fused; k_fused_ring runs it for
// a sequence of batches).  bar_base / epoch: this batch's grid-barrier base and
// epoch; stage_tables: copy the T-tables into shared memory first (a ring's
// later batches find them there).
template <bool MERGED>
__device__ __forceinline__ void fused_body(const DevTable &T, const DevWork &W, const BatchArgs &B,
                                           uint32_t ppc, uint32_t bar_base, uint32_t epoch,
                                           bool stage_tables)
{
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t n_sa = T.n_sa;
    unsigned long long *tr = W.trace ? W.trace + (size_t)blockIdx.x * 8u : nullptr;
    if (tr && tid == 0) tr[0] = gtimer();

    // layout: tables at the first 64 KB-aligned shared address >= base + sizeof(Lo)
    const uint32_t sb = smem_u32(smem);
    const uint32_t toff = (0x10000u - (sb & 0xffffu)) & 0xffffu;
    uint32_t lo_off = 0;
    if (toff < sizeof(FusedLo)) {
        if (toff + AES_TABLE_BYTES + sizeof(FusedHi) + sizeof(FusedLo) > F_SMEM) __trap();
        lo_off = toff + AES_TABLE_BYTES + (uint32_t)sizeof(FusedHi);   // e.g. base 0: after Hi
    }
    uint8_t *tabs = smem + toff;
    FusedLo &L = *reinterpret_cast<FusedLo *>(smem + lo_off);
    FusedHi &H = *reinterpret_cast<FusedHi *>(smem + toff + AES_TABLE_BYTES);
    const uint32_t lane4r = (lane * 4u) | (smem_u32(tabs) & 0xffff0000u);

#if NBA_SA_PREFETCH
    // warm L2 with the SA table (SA lines and counters) while the prologue
    // runs: each CTA prefetches a slice of the 128-byte lines
    {
        const uint32_t nl_sal = T.n_sa;                        // one line per SA
        const uint32_t nl = nl_sal + ((T.n_sa * 4u + 127u) >> 7);
        for (uint32_t l = blockIdx.x * blockDim.x + tid; l < nl; l += gridDim.x * blockDim.x)
            prefetch_l2(l < nl_sal ? reinterpret_cast<const uint8_t *>(T.sal + (size_t)l * SAL_U4)
                                   : reinterpret_cast<const uint8_t *>(T.seq) + 128u * (l - nl_sal));
    }
#endif
    const uint32_t p_begin = blockIdx.x * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    // merged prologue: the packet metadata loads are issued before the table
    // staging so their DRAM latency overlaps it
    uint32_t pre_sa = INVALID_SA, pre_D = 0, pre_inoff = 0, pre_outoff = 0;
    if (MERGED && p_begin + tid < p_end) {
        pre_D = B.in_len[p_begin + tid];
        pre_inoff = B.in_off[p_begin + tid];
        pre_outoff = B.out_off[p_begin + tid];
        pre_sa = B.sa_idx ? B.sa_idx[p_begin + tid]
                          : flow_lookup_one(B.flow_table, B.flow_mask, B.in_buf + pre_inoff, pre_D);
    }
    // the SA counter this warp's row scan will start from (only that scan
    // writes it, after the grid barrier)
    uint32_t old0 = 0;
    if (MERGED) old0 = scan_first_old(T, blockIdx.x * (F_THREADS / 32u) + warp,
                                      gridDim.x * (F_THREADS / 32u), gridDim.x, lane);
    if (stage_tables) tables_stage(tabs, T, &L.tbar, true);   // waited for before the first lookup
    if (tr && tid == 0) tr[2] = gtimer();
    if (tid < 4) L.cnt[tid] = 0ull;
    if (tid < NBINS) L.bins[tid] = 0;   // re-zeroed after each use (length_sort)
    if (MERGED) {
        for (uint32_t k = tid; k < 2u * F_SUPER; k += F_THREADS) {
            L.hkey[k] = INVALID_SA;
            L.hmask[k] = 0;
        }
    }
    __syncthreads();

    static_assert(F_SUPER <= F_THREADS, "one packet per thread in the metadata phase");
    uint32_t c_ok = 0, c_drop = 0, c_in = 0, c_out = 0;

    if constexpr (MERGED) {
        // ---- one super-round; thread j <-> packet p_begin + j ----------------
        constexpr uint32_t NW = F_THREADS / 32u;
        const uint32_t G = gridDim.x, cta = blockIdx.x;
        const uint32_t cnt_pk = p_end > p_begin ? p_end - p_begin : 0u;
        const uint32_t j = tid;
        const bool cand = j < cnt_pk && pre_sa < n_sa && pre_D >= MIN_D && pre_D <= MAX_D;
        const uint32_t bin = hmac_bin(cand, esp_C(pre_D));
        if (j < cnt_pk) {
            L.sa[j] = pre_sa;
            L.info[j] = cand ? (pre_D | INFO_OK) : 0u;
            L.inoff[j] = pre_inoff;
            L.outoff[j] = pre_outoff;
            // the lane reads the payload after the barrier: DRAM -> L2 now
            if (cand) prefetch_bytes(B.in_buf + pre_inoff, min(64u, pre_D));
        }
        warp_agg_add(L.bins, bin, j < cnt_pk);
        // 1. CTA-local ranks and per-SA counts (the prologue's tile part)
        const uint32_t rank = merged_local_rank(W, L, cand ? pre_sa : INVALID_SA);
        if (j < cnt_pk) L.seq[j] = rank;
        if (tr && tid == 0) tr[4] = gtimer();
        // 2. lane order: longest packets first (seq-overflow drops keep their bin)
        length_sort(L, j, cnt_pk, bin);   // ends with __syncthreads: counts written
        grid_arrive(&W.ctl[CTL_BAR_MONO]);
        if (tr && tid == 0) tr[1] = gtimer();
        // 3. between arrival and wait: issue the loads of the lane's SA line and
        //    TOS byte (used after the barrier)
        uint32_t pos;
        const bool have = lane_position(L, cnt_pk, pos);
        const uint32_t pk = have ? L.perm[pos] : 0u;
        const uint32_t info = have ? L.info[pk] : 0u;
        const uint32_t sa_me = (info & INFO_OK) ? L.sa[pk] : INVALID_SA;
        const uint32_t inoff = have ? L.inoff[pk] : 0u;
        PktPre pp = {};
        if (sa_me != INVALID_SA) {
            pp = load_pkt_pre(T, B.in_buf, sa_me, inoff, true, 0u);
            tables_bulk_wait(&L.tbar, 0u);
            if (!NBA_EXPAND_MID) expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
        }
        grid_wait(&W.ctl[CTL_BAR_MONO], bar_base + G);
        if (blockIdx.x == 0 && tid == 0) {
            W.ctl[CTL_BAR_BASE] = bar_base + G;
            W.ctl[CTL_EPOCH] = epoch;
        }
        if (tr && tid == 0) tr[5] = gtimer();
        // 4. row scans publish epoch-tagged bases; each packet polls its own
        //    (SA, CTA) entry
        scan_all_columns<true>(T, W, cta * NW + warp, G * NW, G, lane, epoch, true, old0);
        if (tr && tid == 0) tr[6] = gtimer();
        // round keys into shared memory: after the scans (nothing before the
        // barrier waits for the SA line) and while the bases propagate
        if (NBA_EXPAND_MID && sa_me != INVALID_SA) expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
        __syncwarp();
        // 5. sequence numbers: thread j polls the published base of its packet's
        //    (SA, CTA) entry; all polls end before any lane starts its packet
        //    (measured: letting each warp start after its own polls leaves
        //    stragglers whose polls end only with other CTAs' lane phases)
        if (cand) {
            const unsigned long long *pb = &W.hbase[(size_t)pre_sa * G + cta];
            unsigned long long v = ld_relaxed_u64(pb);
            while ((uint32_t)(v >> 33) != epoch) {
                if (NBA_POLL_NS) __nanosleep(NBA_POLL_NS);
                v = ld_relaxed_u64(pb);
            }
            const unsigned long long q = (v & ((1ull << 33) - 1ull)) + 1ull + rank;
            L.seq[j] = q <= 0xffffffffull ? (uint32_t)q : 0u;   // RFC 4303 §3.3.3: never cycle
        }
        __syncthreads();
        if (tr && lane == 0) atomicMax(&tr[7], gtimer());
        const uint32_t q32 = (sa_me != INVALID_SA) ? L.seq[pk] : 0u;
        const bool ok = q32 != 0u;   // a valid sequence number is never 0
        // 6. the lane's packet
#ifndef NBA_PROLOGUE_ONLY      // debug A/B: 1 skips the lane phase (timing of the prologue alone)
#define NBA_PROLOGUE_ONLY 0
#endif
        if (have && !NBA_PROLOGUE_ONLY) {
            const uint32_t pkt = p_begin + pk;
            if (ok) {
                esp_packet(T, B, L, H, lane4r, tid, sa_me, info, q32, inoff, L.outoff[pk], pp,
                           (tr && blockIdx.x == 0 && (pos == 0 || pos == cnt_pk - 1u))
                               ? W.trace + 148 * 8 + 8 + (pos == 0 ? 0 : 8) : nullptr);
                const uint32_t Dp = info & 0x7ffu;
                const uint32_t Lp = 48u + esp_C(Dp);
                B.out_len[pkt] = (uint16_t)Lp;
                c_ok++;
                c_in += Dp;
                c_out += Lp;
            } else {
                B.out_len[pkt] = 0;
                c_drop++;
            }
        }
        if (tr && lane == 0) {
            const unsigned long long now = gtimer();
            atomicMax(&tr[3], now);
            if (blockIdx.x == 0) W.trace[W.trace_pro + 24u + warp] = now;   // CTA 0, per warp
        }
    } else {
    for (uint32_t base = p_begin; base < p_end; base += F_SUPER) {
        const uint32_t cnt_pk = min((uint32_t)F_SUPER, p_end - base);
        // ---- 1. metadata (thread j <-> packet base + j) ---------------------
        const uint32_t j = tid;
        const uint32_t i = base + j;
        // 1a. everything that does not depend on the prologue (overlaps it under
        //     programmatic dependent launch on the first round)
        uint32_t sa = INVALID_SA, D = 0, inoff = 0, tos = 0;
        bool cand = false;
        if (j < cnt_pk) {
            sa = B.sa_idx[i];
            D = B.in_len[i];
            inoff = B.in_off[i];
            L.outoff[j] = B.out_off[i];
            cand = sa < n_sa && D >= MIN_D && D <= MAX_D;
            if (cand) tos = B.in_buf[inoff + 1];
        }
        if (base == p_begin) {
            // Programmatic dependent launch: the prologue kernel's outputs (ranks,
            // per-SA prefixes, seq_prev) are complete and visible after this.
            asm volatile("griddepcontrol.wait;" ::: "memory");
        }
        // 1b. sequence number, drop decision, length bin
        uint32_t bin = NBINS - 1;
        if (j < cnt_pk) {
            uint32_t info = 0, q32 = 0;
            if (cand) {
                const unsigned long long q =
                    (unsigned long long)T.seq_prev[sa] + 1ull +
                    W.hpfx[(size_t)sa * ((B.n + PTILE - 1) / PTILE) + i / PTILE] + W.lrank[i];
                if (q <= 0xffffffffull) {   // RFC 4303 §3.3.3: never cycle
                    q32 = (uint32_t)q;
                    info = D | (tos << 16) | INFO_OK;
                    bin = hmac_bin(true, esp_C(D));
                }
            }
            L.sa[j] = sa;
            L.seq[j] = q32;
            L.info[j] = info;
            L.inoff[j] = inoff;
        }
        warp_agg_add(L.bins, bin, j < cnt_pk);
        length_sort(L, j, cnt_pk, bin);   // also publishes the T-tables on the first round
        if (tr && tid == 0 && base == p_begin) tr[1] = gtimer();

        // ---- 2. one lane per packet, length-sorted so a warp's lanes do equal
        // work; the longest packets go to the LOWEST warps (measured on B200:
        // -2% at IMIX vs the highest warps, tools/ab_variants.py)
        {
            uint32_t pos;
            const bool have = lane_position(L, cnt_pk, pos);
            const uint32_t pk = have ? L.perm[NBA_LONG_HIGH ? cnt_pk - 1u - pos : pos] : 0u;
            const uint32_t info = have ? L.info[pk] : 0u;
            const uint32_t pkt = base + pk;
            const uint32_t sa_me = (info & INFO_OK) ? L.sa[pk] : INVALID_SA;
            if (tr && tid == 0) tr[7] = gtimer();
            if (!have) {
            } else if (info & INFO_OK) {
                PktPre pp = load_pkt_pre(T, B.in_buf, sa_me, L.inoff[pk], false, (info >> 16) & 0xffu);
                tables_bulk_wait(&L.tbar, 0u);
                expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
                esp_packet(T, B, L, H, lane4r, tid, sa_me, info, L.seq[pk], L.inoff[pk],
                           L.outoff[pk], pp,
                           (tr && blockIdx.x == 0 && (pos == 0 || pos == cnt_pk - 1u))
                               ? W.trace + 148 * 8 + 8 + (pos == 0 ? 0 : 8) : nullptr);
                const uint32_t Dp = info & 0x7ffu;
                const uint32_t Lp = 48u + esp_C(Dp);
                B.out_len[pkt] = (uint16_t)Lp;
                c_ok++;
                c_in += Dp;
                c_out += Lp;
            } else {
                B.out_len[pkt] = 0;
                c_drop++;
            }
        }
        if (tr && lane == 0) atomicMax(&tr[3], gtimer());
        __syncthreads();   // shared metadata is reused by the next super-round
    }
    }
    tables_bulk_wait(&L.tbar, 0u);   // no bulk copy in flight past here (threads without packets)
    // counters: warp sums, then one 64-bit atomic per CTA and counter
    const uint32_t s0 = __reduce_add_sync(0xffffffffu, c_ok);
    const uint32_t s1 = __reduce_add_sync(0xffffffffu, c_drop);
    const uint32_t s2 = __reduce_add_sync(0xffffffffu, c_in);
    const uint32_t s3 = __reduce_add_sync(0xffffffffu, c_out);
    if (lane == 0) {
        atomicAdd(&L.cnt[0], (unsigned long long)s0);
        atomicAdd(&L.cnt[1], (unsigned long long)s1);
        atomicAdd(&L.cnt[2], (unsigned long long)s2);
        atomicAdd(&L.cnt[3], (unsigned long long)s3);
    }
    __syncthreads();
    if (tid < 4 && L.cnt[tid]) atomicAdd(&W.counters[tid], L.cnt[tid]);
    if (tid == 4 && blockIdx.x == 0) atomicAdd(&W.counters[4], 1ull);
    if (tr && tid == 0) atomicMax(W.trace + W.trace_pro + 48u, gtimer());   // CTA end
}

template <bool MERGED>
__global__ void __launch_bounds__(F_THREADS, 1)
k_fused(DevTable T, DevWork W, BatchArgs B, uint32_t ppc, uint32_t bar_base_h, uint32_t epoch_h)
{
    // one-kernel path: barrier base and batch epoch from the device (read by
    // every thread before its CTA arrives at the grid barrier; CTA 0 advances
    // them after the barrier, when every CTA has read them)
    uint32_t bar_base = bar_base_h, epoch = epoch_h;
    if (MERGED) {
        bar_base = *reinterpret_cast<volatile uint32_t *>(&W.ctl[CTL_BAR_BASE]);
        epoch = (*reinterpret_cast<volatile uint32_t *>(&W.ctl[CTL_EPOCH]) % 0x7fffffffu) + 1u;
    }
    fused_body<MERGED>(T, W, B, ppc, bar_base, epoch, true);
}

// A batch ring as ONE persistent launch (nba_ipsec_ring_run): the grid (one
// CTA per SM) walks n_batches batches, slot bi mod n_slots, keeping the
// T-tables in shared memory; a CTA that finishes batch bi starts bi + 1's
// metadata phase while the others finish, and waits at that batch's grid
// barrier.  The per-(SA, CTA) count matrix alternates between two buffers by
// batch parity: batch bi's row scans re-zero buffer bi & 1 after every CTA
// passed barrier bi, and batch bi + 2 writes it only after barrier bi + 1.
__global__ void __launch_bounds__(F_THREADS, 1)
k_fused_ring(DevTable T, DevWork W, const BatchArgs *slots, RingRun R, uint16_t *hist_b)
{
    const uint32_t n_slots = R.n_slots, n_batches = R.n_batches;
    if (R.ts && blockIdx.x == 0 && threadIdx.x == 0) R.ts[0] = gtimer();
    const uint32_t base0 = *reinterpret_cast<volatile uint32_t *>(&W.ctl[CTL_BAR_BASE]);
    const uint32_t ep0 = *reinterpret_cast<volatile uint32_t *>(&W.ctl[CTL_EPOCH]);
    const uint32_t G = gridDim.x;
    for (uint32_t bi = 0; bi < n_batches; bi++) {
        const BatchArgs B = slots[(R.first + bi) % n_slots];
        DevWork Wb = W;
        if (bi & 1u) Wb.hist16 = hist_b;
        const uint32_t epoch = ((ep0 + bi) % 0x7fffffffu) + 1u;
        fused_body<true>(T, Wb, B, fused_ppc(B.n, G), base0 + bi * G, epoch, bi == 0);
        __syncthreads();   // shared memory is reused by the next batch
        if (R.ts && threadIdx.x == 0) atomicMax(&R.ts[1u + bi], gtimer());
    }
}

// ------------------------------------------- software-pipelined batch ring
// k_fused_ring_pipe: the ring with warp roles.  Warps 0..13 ("lanes") carry
// batch k's packets, one per lane (ppc <= 448); warps 14..15 ("prologue")
// meanwhile prepare batch k+1 for this CTA -- metadata, CTA-local stable
// per-SA ranks (rounds of 64 packets in index order through a shared hash of
// running counts), the per-(SA, CTA) counts, the length order -- arrive at
// batch k+1's grid barrier, run their share of the row scans (two warps per
// CTA) and poll the published bases into L.seq.  The lanes copy their
// packet's fields into registers first (named barrier 2), so one set of
// per-packet shared arrays serves both batches; each lane expands its own
// round keys.  Same arithmetic and the same results as the other paths; the
// count matrix alternates between two buffers by batch parity as in
// k_fused_ring.
#ifndef NBA_PIPE_EARLY_KEYS   // pipelined ring: SA line + round keys before the scans / polls:
#define NBA_PIPE_EARLY_KEYS 2 // 1 always, 0 never, 2 per batch (long or length-divergent)
#endif
#ifndef NBA_PIPE_PSCAN        // pipelined ring: the prologue warps also run the row scans:
#define NBA_PIPE_PSCAN 0      // 0 never, 1 always, 2 when most CTAs vote the batch long,
#endif                        // 3 always + the prologue warps poll the bases too (the next
                              //   batch's sequence numbers are ready when it starts)
#ifndef NBA_PIPE_LPT          // pipelined ring: LPT placement of the runs (1) or run r -> warp r
#define NBA_PIPE_LPT 1
#endif
#ifndef NBA_RING_TRACE        // debug variant: per-(batch, CTA) phase stamps into RingRun::ts
#define NBA_RING_TRACE 0      //   (tools/ring_trace.py; [n_batches][G][8] globaltimer ns)
#endif
#if NBA_RING_TRACE
#define RTR(bi, k) (R.ts ? R.ts + ((size_t)(bi) * gridDim.x + blockIdx.x) * 16u + (k) : nullptr)
#endif

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    return v;   // lane 0
}

// The prologue warps' share of the row scans (rows slot, slot + nslots, ...),
// four rows at a time: 8 lanes per row, each lane owning CPL consecutive
// columns (G <= 8 x CPL = 160 CTAs).  A lane loads its columns' counts (all
// loads in flight together), sums them in registers, and one 3-step shuffle
// scan across the row's 8 lanes gives each lane its starting prefix: ONE
// memory round trip and a short shuffle chain per four rows, instead of a
// 5 x 5-step shuffle chain per row.  Same results as scan_all_columns.
__device__ __forceinline__ void pipe_scan_rows(const DevTable &T, const DevWork &W, uint32_t slot,
                                               uint32_t nslots, uint32_t G, uint32_t lane,
                                               uint32_t epoch)
{
    constexpr uint32_t CPL = 20;                 // columns per lane (8 lanes per row)
    const uint32_t r = lane >> 3, q = lane & 7u, c0 = q * CPL;
    for (uint32_t g = 0; slot + g * 4u * nslots < T.n_sa; g++) {
        const uint32_t sa = slot + (4u * g + r) * nslots;
        const bool ok = sa < T.n_sa;
        uint16_t *col = W.hist16 + (size_t)(ok ? sa : 0u) * G;
        const uint32_t old = (ok && q == 0) ? T.seq[sa] : 0u;
        uint32_t h[CPL];
#pragma unroll
        for (uint32_t k = 0; k < CPL; k++) h[k] = (ok && c0 + k < G) ? (uint32_t)__ldcg(&col[c0 + k]) : 0u;
        uint32_t sum = 0;
#pragma unroll
        for (uint32_t k = 0; k < CPL; k++) sum += h[k];
        uint32_t x = sum;                        // inclusive scan over the row's 8 lanes
#pragma unroll
        for (uint32_t o = 1; o < 8u; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o, 8);
            if (q >= o) x += y;
        }
        const uint32_t tot = __shfl_sync(0xffffffffu, x, 7, 8);
        const uint32_t old_r = __shfl_sync(0xffffffffu, old, 0, 8);
        if (ok) {
            unsigned long long run = (unsigned long long)old_r + (x - sum);
#pragma unroll
            for (uint32_t k = 0; k < CPL; k++) {
                if (c0 + k < G) {
                    st_relaxed_u64(&W.hbase[(size_t)sa * G + c0 + k], ((unsigned long long)epoch << 33) | run);
                    if (h[k]) col[c0 + k] = 0;   // re-arm for the next batch of this parity
                }
                run += h[k];
            }
            if (q == 0) {
                T.seq_prev[sa] = old_r;
                const uint32_t room = 0xffffffffu - old_r;
                T.seq[sa] = old_r + (tot < room ? tot : room);
            }
        }
    }
}

// The packet metadata of this prologue thread (packets j = r * 64 + pt of the
// CTA's range, r < 7), all loads issued together.
constexpr uint32_t PR = PIPE_MAX_PPC / PIPE_P;                      // 7 rounds
struct PipeMeta {
    uint32_t D[PR], S[PR], I[PR], O[PR];
};

__device__ __forceinline__ void pipe_load_meta(const BatchArgs &B, uint32_t ppc, uint32_t pt, PipeMeta &m)
{
    const uint32_t p_begin = blockIdx.x * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {
        const uint32_t j = r * PIPE_P + pt;
        const uint32_t i = p_begin + j;
        m.D[r] = j < cnt ? B.in_len[i] : 0u;
        m.S[r] = j < cnt ? B.sa_idx[i] : INVALID_SA;
        m.I[r] = j < cnt ? B.in_off[i] : 0u;
        m.O[r] = j < cnt ? B.out_off[i] : 0u;
    }
}

// L2 prefetch of a batch's metadata lines for this CTA (in_len, sa_idx,
// in_off, out_off of its packet range) by the 64 prologue threads: issued two
// batches ahead, so the prologue's metadata loads hit L2 (the ring's slots
// rotate through more than the L2, the arrays are DRAM-cold otherwise).
__device__ __forceinline__ void pipe_prefetch_meta(const BatchArgs &B, uint32_t ppc, uint32_t pt)
{
    const uint32_t p_begin = blockIdx.x * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    if (p_end <= p_begin) return;
    const uint32_t cnt = p_end - p_begin;
    // lines of the four arrays: 2-byte and 4-byte elements, <= 448 packets
    const uint32_t l16 = (2u * cnt + 127u) / 128u + 1u, l32 = (4u * cnt + 127u) / 128u + 1u;
    const uint32_t tot = l16 + 3u * l32;
    for (uint32_t k = pt; k < tot; k += PIPE_P) {
        const uint8_t *a;
        if (k < l16) {
            a = reinterpret_cast<const uint8_t *>(B.in_len + p_begin) + 128u * k;
            if (a >= reinterpret_cast<const uint8_t *>(B.in_len + p_end)) continue;
        } else {
            const uint32_t q = (k - l16) / l32, m = (k - l16) % l32;
            const uint32_t *base = q == 0 ? B.sa_idx : q == 1 ? B.in_off : B.out_off;
            a = reinterpret_cast<const uint8_t *>(base + p_begin) + 128u * m;
            if (a >= reinterpret_cast<const uint8_t *>(base + p_end)) continue;
        }
        prefetch_l2(a);
    }
}

#ifndef NBA_PIPE_DIRECT       // pipelined ring: per-SA counts in arrays indexed by the SA
#define NBA_PIPE_DIRECT 0     //   (n_sa <= 1024: no hash probing; measured slower under the lanes' load) instead of the hash
#endif
constexpr uint32_t PIPE_DIRECT_MAX_SA = 2u * F_SUPER;              // 1024 (the hash arrays' size)

// Prologue of one batch by the 64 prologue threads (pt = 0..63) of this CTA.
__device__ __forceinline__ void pipe_prologue(const DevTable &T, const DevWork &W, const BatchArgs &B,
                                              uint32_t ppc, uint32_t bar_target, uint32_t epoch,
                                              FusedLo &L, uint32_t pt, uint32_t parity,
                                              const PipeMeta &m, unsigned long long *tr = nullptr)
{
    const uint32_t G = gridDim.x, cta = blockIdx.x, n_sa = T.n_sa;
    const uint32_t lane = pt & 31u, pw = pt >> 5;
    const uint32_t p_begin = cta * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
    const uint32_t rounds = (cnt + PIPE_P - 1u) / PIPE_P;
    const bool direct = NBA_PIPE_DIRECT && n_sa <= PIPE_DIRECT_MAX_SA;
    // 1. metadata (loaded by pipe_load_meta), validity, length bins (counts)
    uint32_t st_sum = 0, st_max = 0;   // AES steps of the valid packets
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {
        const uint32_t j = r * PIPE_P + pt;
        uint32_t bin = NBINS - 1;
        if (j < cnt) {
            const bool cand = m.S[r] < n_sa && m.D[r] >= MIN_D && m.D[r] <= MAX_D;
            const uint32_t stp = cand ? (esp_C(m.D[r]) + 63u) >> 6 : 0u;
            st_sum += stp;
            st_max = max(st_max, stp);
            L.sa[j] = m.S[r];
            L.info[j] = cand ? (m.D[r] | INFO_OK) : 0u;
            L.inoff[j] = m.I[r];
            L.outoff[j] = m.O[r];
            bin = hmac_bin(cand, esp_C(m.D[r]));
            if (cand) prefetch_bytes(B.in_buf + m.I[r], min(64u, m.D[r]));   // the lane reads it next round
        }
        if (r < rounds) warp_agg_add(L.bins, bin, j < cnt);
    }
    st_sum = __reduce_add_sync(0xffffffffu, st_sum);
    st_max = __reduce_max_sync(0xffffffffu, st_max);
    if (pt == 0) {
        L.pstat[0] = st_sum;
        L.pstat[1] = st_max;
    }
    bar_sync_n(1, PIPE_P);
    if (tr && pt == 0) tr[8] = gtimer();
    if (pt == 32) {     // the second prologue warp adds its share
        L.pstat[0] += st_sum;
        L.pstat[1] = max(L.pstat[1], st_max);
    }
    // 2. stable CTA-local ranks: prologue warp w ranks its half of the packets
    //    (rounds of 32 in index order) with its own running count per SA
    //    (direct: arrays indexed by the SA -- warp 0 L.hmask, warp 1 cnt1 --;
    //    else per slot of the CTA's SA hash), concurrently; warp 1's ranks then
    //    add warp 0's final count of the SA
    uint32_t *cnt1 = &L.aux0[0];                 // aux0 | aux1: 1024 counts (outbound only)
    const uint32_t half = ((cnt + 1u) / 2u + 31u) & ~31u;
    const uint32_t j0 = pw ? half : 0u, j1 = pw ? cnt : min(cnt, half);
    {
        uint32_t *cw = pw ? cnt1 : L.hmask;
        for (uint32_t jb = j0; jb < j1; jb += 32u) {
            const uint32_t j = jb + lane;
            const bool act = j < j1 && (L.info[j] & INFO_OK);
            const uint32_t s = act ? L.sa[j] : INVALID_SA;
            const uint32_t peers = __match_any_sync(0xffffffffu, s);
            const uint32_t leader = __ffs(peers) - 1;
            uint32_t base = 0, slot = s;
            if (act && lane == leader) {
                if (!direct) {
                    slot = (s * 0x9E3779B1u) >> 22;          // 1024 slots
                    while (true) {
                        const uint32_t old = atomicCAS(&L.hkey[slot], INVALID_SA, s);
                        if (old == INVALID_SA || old == s) break;
                        slot = (slot + 1u) & (2u * F_SUPER - 1u);
                    }
                }
                base = cw[slot];
                cw[slot] = base + (uint32_t)__popc(peers);
            }
            base = __shfl_sync(0xffffffffu, base, leader);
            if (!direct) slot = __shfl_sync(0xffffffffu, slot, leader);
            if (j < j1) {
                L.seq[j] = act ? base + (uint32_t)__popc(peers & lanemask_lt()) : 0u;
                if (pw && !direct) L.perm[j] = (uint16_t)slot;     // (perm is rebuilt in step 3)
            }
        }
        bar_sync_n(1, PIPE_P);
        if (pw) {
            for (uint32_t j = j0 + lane; j < j1; j += 32u)
                if (L.info[j] & INFO_OK) L.seq[j] += L.hmask[direct ? L.sa[j] : L.perm[j]];
        }
        bar_sync_n(1, PIPE_P);
        if (tr && pt == 0) tr[9] = gtimer();
    }
    // 3. this CTA's per-SA counts -> count matrix (nonzero only) and the
    //    counters cleared for the next batch: direct -- the SA's last packet in
    //    the CTA (rank = count - 1) writes it; hash -- a sweep over the slots.
    //    Length order: exclusive scan of the bins, positions, bins re-zeroed;
    //    a batch whose packets all share one bin keeps index order.
    uint32_t owner = 0;                          // direct: rounds whose packet is its SA's last
    if (direct) {
#pragma unroll
        for (uint32_t r = 0; r < PR; r++) {
            const uint32_t j = r * PIPE_P + pt;
            if (j < cnt && (L.info[j] & INFO_OK)) {
                const uint32_t s = L.sa[j];
                const uint32_t tot = L.hmask[s] + cnt1[s];
                if (L.seq[j] + 1u == tot) {
                    W.hist16[(size_t)s * G + cta] = (uint16_t)tot;
                    owner |= 1u << r;            // clears the counters after the barrier
                }
            }
        }
    } else {
        for (uint32_t k = pt; k < 2u * F_SUPER; k += PIPE_P) {
            const uint32_t s = L.hkey[k];
            if (s != INVALID_SA) {
                W.hist16[(size_t)s * G + cta] = (uint16_t)(L.hmask[k] + cnt1[k]);
                cnt1[k] = 0u;
                L.hkey[k] = INVALID_SA;
                L.hmask[k] = 0u;
            }
        }
    }
    bool one_bin = false;
    if (pw == 0) {
        const uint32_t cb = L.bins[lane];
        one_bin = __any_sync(0xffffffffu, cb == cnt);
        uint32_t x = cb;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= (uint32_t)o) x += y;
        }
        L.bins[lane] = x - cb;
        if (lane == 0) L.pstat[2] = one_bin ? 4u : 0u;     // bit 2: one length bin
    }
    bar_sync_n(1, PIPE_P);
    if (tr && pt == 0) tr[10] = gtimer();
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {          // every total was read: clear for the next batch
        if ((owner >> r) & 1u) {
            const uint32_t s = L.sa[r * PIPE_P + pt];
            L.hmask[s] = 0u;
            cnt1[s] = 0u;
        }
    }
    one_bin = NBA_PIPE_ONEBIN && (L.pstat[2] & 4u) != 0u;
    for (uint32_t r = 0; r < rounds; r++) {
        const uint32_t j = r * PIPE_P + pt;
        if (one_bin) {                           // counting sort of one bin = index order
            if (j < cnt) L.perm[j] = (uint16_t)j;
            continue;
        }
        const uint32_t info = j < cnt ? L.info[j] : 0u;
        const uint32_t bin = hmac_bin((info & INFO_OK) != 0u, esp_C(info & 0x7ffu));
        const uint32_t pos = warp_agg_add(L.bins, bin, j < cnt);
        if (j < cnt) L.perm[pos] = (uint16_t)j;
    }
    bar_sync_n(1, PIPE_P);                      // count-matrix writes done, bins read
    if (tr && pt == 0) tr[11] = gtimer();
    if (pt < NBINS) L.bins[pt] = 0u;
    if (pt == 0) {
        // round keys before the scans / polls (their latency overlaps) pays for
        // long or length-divergent batches; for uniform short ones after
        // (measured: 64 B 23.5 vs 24.1 us, IMIX 96.8 vs 90.4, 1514 B 193.7 vs 192.3)
        const uint32_t sum = L.pstat[0], mx = L.pstat[1], nv = cnt ? cnt : 1u;
        L.pstat[2] = (L.pstat[2] & 4u) | ((mx * nv > 2u * sum || sum >= 8u * nv) ? 1u : 0u);
    }
    if (pw == 0 && !NBA_PIPE_LPT) {
        if (lane < PIPE_LANE_WARPS) L.wrun[lane] = (uint8_t)lane;   // run r -> warp r
    } else if (pw == 0) {
        // runs of 32 sorted positions -> lane warps, longest first onto the least
        // loaded sub-partition (warp w issues on w mod 4; lane warps 0..13, so
        // sub-partitions 0 / 1 hold 4 of them and 2 / 3 hold 3), as length_sort
        const uint32_t nruns = (cnt + 31u) / 32u;
        uint32_t cost = 0;
        if (lane < nruns) {
            const uint32_t info = L.info[L.perm[32u * lane]];
            const uint32_t C = esp_C(info & 0x7ffu);
            cost = (info & INFO_OK) ? 8u * (esp_nsha_inner(C) + 1u) + 3u * ((C + 15u) >> 4) : 1u;
        }
        const uint32_t c0 = __shfl_sync(0xffffffffu, cost, 0);
        uint32_t mine = lane < nruns ? lane : 0xffu;      // equal costs: run r -> warp r
        if (!__all_sync(0xffffffffu, lane >= nruns || cost == c0))
            mine = lpt_place(cost, nruns, lane, 4u, 4u, 3u, 3u);
        if (lane < PIPE_LANE_WARPS) L.wrun[lane] = (uint8_t)mine;
    }
    // 4. arrive at this batch's grid barrier (the whole CTA waits for it at
    //    the start of the batch's iteration; the arrival releases the count
    //    matrix writes above, ordered by the named barrier)
#if NBA_PIPE_PSCAN == 2
    // this CTA's vote: a long batch (mean >= 8 AES steps) lets the prologue
    // warps run the row scans too (published before the arrival releases it)
    if (pt == 0) {
        const uint32_t nv = cnt ? cnt : 1u;
        const unsigned long long vote = L.pstat[0] >= 8u * nv ? 1ull : 0ull;
        W.pvote[(size_t)parity * G + cta] = ((unsigned long long)epoch << 1) | vote;
    }
#endif
    if (tr && pt == 0) tr[12] = gtimer();
    if (pt == 0)
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&W.ctl[CTL_BAR_MONO]) : "memory");
    if (tr && pt == 0) tr[4] = gtimer();   // (trace variant: tr = this iteration's stamps)
#if NBA_PIPE_PSCAN
    // and, once every CTA arrived, this CTA's share of the row scans (two
    // warps) -- always (PSCAN 1), or when most CTAs voted "long" (PSCAN 2: the
    // same count of the same complete votes in every CTA, so all agree)
    if (pt == 0) {
        uint32_t v;
        while (true) {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&W.ctl[CTL_BAR_MONO]) : "memory");
            if ((int)(v - bar_target) >= 0) break;
            __nanosleep(128);
        }
    }
    bar_sync_n(1, PIPE_P);
    if (tr && pt == 0) tr[1] = gtimer();
    bool pscan = true;
#if NBA_PIPE_PSCAN == 2
    {
        uint32_t longs = 0;
#pragma unroll
        for (uint32_t u = 0; u < 5u; u++) {
            const uint32_t c = 32u * u + lane;
            const unsigned long long e = c < G ? ld_relaxed_u64(&W.pvote[(size_t)parity * G + c]) : 0ull;
            longs += __popc(__ballot_sync(0xffffffffu, c < G && (uint32_t)(e >> 1) == epoch && (e & 1ull)));
        }
        pscan = 2u * longs > G;
        if (pt == 0) L.pstat[2] |= pscan ? 2u : 0u;    // bit 1: the CTA skips its scans
    }
#endif
    if (pscan) pipe_scan_rows(T, W, cta * 2u + pw, G * 2u, G, lane, epoch);
    if (tr && pt == 0) tr[2] = gtimer();
#if NBA_PIPE_PSCAN == 3
    // the sequence numbers of this CTA's packets: every poll issued before any
    // is re-tried (one memory round trip when the bases are already published)
    {
        unsigned long long v[PR];
        uint32_t sa_r[PR];
#pragma unroll
        for (uint32_t r = 0; r < PR; r++) {
            const uint32_t j = r * PIPE_P + pt;
            const bool ok = j < cnt && (L.info[j] & INFO_OK);
            sa_r[r] = ok ? L.sa[j] : INVALID_SA;
            v[r] = ok ? ld_relaxed_u64(&W.hbase[(size_t)sa_r[r] * G + cta]) : 0ull;
        }
#pragma unroll
        for (uint32_t r = 0; r < PR; r++) {
            const uint32_t j = r * PIPE_P + pt;
            if (j >= cnt) continue;
            uint32_t q32 = 0;
            if (sa_r[r] != INVALID_SA) {
                const unsigned long long *pb = &W.hbase[(size_t)sa_r[r] * G + cta];
                while ((uint32_t)(v[r] >> 33) != epoch) v[r] = ld_relaxed_u64(pb);
                const unsigned long long q = (v[r] & ((1ull << 33) - 1ull)) + 1ull + L.seq[j];
                q32 = q <= 0xffffffffull ? (uint32_t)q : 0u;   // RFC 4303 §3.3.3: never cycle
            }
            L.seq[j] = q32;
        }
        if (tr && (pt & 31u) == 0) atomicMax(&tr[7], gtimer());
    }
#endif
#endif
}

// The batch's barrier wait, row scans and published bases, by the whole CTA
// (thread j <-> packet j): L.seq[j] turns from the CTA rank into the ESP
// sequence number (0: no number, the packet is dropped).
__device__ __forceinline__ void pipe_sequence(const DevTable &T, const DevWork &W, const BatchArgs &B,
                                              uint32_t ppc, uint32_t bar_target, uint32_t epoch,
                                              FusedLo &L, unsigned long long *tr = nullptr)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x;
    constexpr uint32_t NW = F_THREADS / 32u;
    if (NBA_PIPE_PSCAN == 3) return;   // the prologue warps numbered the packets already
    if (tid == 0) {
        uint32_t v;
        while (true) {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&W.ctl[CTL_BAR_MONO]) : "memory");
            if ((int)(v - bar_target) >= 0) break;
        }
        if (tr) tr[1] = gtimer();
    }
    __syncthreads();
    const bool p_scanned = NBA_PIPE_PSCAN == 1 || (NBA_PIPE_PSCAN == 2 && (L.pstat[2] & 2u));
    if (!p_scanned) scan_all_columns<true>(T, W, cta * NW + warp, G * NW, G, lane, epoch, false, 0u);
    const uint32_t p_begin = cta * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
    const uint32_t j = tid;
    if (j < cnt) {
        uint32_t q32 = 0;
        if (L.info[j] & INFO_OK) {
            const unsigned long long *pb = &W.hbase[(size_t)L.sa[j] * G + cta];
            unsigned long long v = ld_relaxed_u64(pb);
            while ((uint32_t)(v >> 33) != epoch) v = ld_relaxed_u64(pb);
            const unsigned long long q = (v & ((1ull << 33) - 1ull)) + 1ull + L.seq[j];
            q32 = q <= 0xffffffffull ? (uint32_t)q : 0u;   // RFC 4303 §3.3.3: never cycle
        }
        L.seq[j] = q32;
    }
    __syncthreads();
    if (tr && tid == 0) tr[2] = gtimer();
}

__global__ void __launch_bounds__(F_THREADS, 1)
k_fused_ring_pipe(DevTable T, DevWork W, const BatchArgs *slots, RingRun R, uint16_t *hist_b)
{
    const uint32_t n_slots = R.n_slots, n_batches = R.n_batches, first = R.first;
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x;
    if (n_batches == 0) return;
    if (!NBA_RING_TRACE && R.ts && cta == 0 && tid == 0) R.ts[0] = gtimer();
    const uint32_t base0 = *reinterpret_cast<volatile uint32_t *>(&W.ctl[CTL_BAR_BASE]);
    const uint32_t ep0 = *reinterpret_cast<volatile uint32_t *>(&W.ctl[CTL_EPOCH]);
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
    tables_stage(tabs, T, &L.tbar, true);   // bulk copy, waited for before the first lookup
    if (tid < NBINS) L.bins[tid] = 0u;
    if (tid == 0) {
        L.stag_ns = 0u;
        L.stag_acc = 0u;
        L.lanes_acc = 0u;
        L.pro_delay = NBA_PIPE_PRO_DELAY0;
    }
    for (uint32_t k = tid; k < PIPE_MAX_PPC; k += F_THREADS) L.tailf[k] = 0u;   // split: ready flags
    for (uint32_t k = tid; k < 2u * F_SUPER; k += F_THREADS) {
        L.hkey[k] = INVALID_SA;
        L.hmask[k] = 0u;
        (&L.aux0[0])[k] = 0u;                     // the prologue's second count array
    }
    __syncthreads();
    const bool isP = tid >= PIPE_MAX_PPC;
    const uint32_t pt = tid - PIPE_MAX_PPC;
    auto epoch_of = [&](uint32_t bi) { return ((ep0 + bi) % 0x7fffffffu) + 1u; };
    auto work_of = [&](uint32_t bi) {
        DevWork Wb = W;
        if (bi & 1u) Wb.hist16 = hist_b;
        return Wb;
    };
    if (isP) {
        if (NBA_PIPE_META_PF && n_batches > 1) {
            const BatchArgs B1 = slots[(first + 1) % n_slots];
            pipe_prefetch_meta(B1, fused_ppc(B1.n, G), pt);
        }
        const BatchArgs B0 = slots[first % n_slots];
        PipeMeta meta;
        pipe_load_meta(B0, fused_ppc(B0.n, G), pt, meta);
#if NBA_RING_TRACE
        if (pt == 0 && R.ts) *RTR(0, 13) = gtimer();      // start-up: batch 0's metadata issued
#endif
        pipe_prologue(T, work_of(0), B0, fused_ppc(B0.n, G), base0 + G, epoch_of(0), L, pt, 0u, meta);
#if NBA_RING_TRACE
        if (pt == 0 && R.ts) *RTR(0, 14) = gtimer();      // start-up: batch 0's prologue done
#endif
    }
#if NBA_RING_TRACE
    if (tid == 0 && R.ts) *RTR(0, 15) = gtimer();          // start-up: kernel start (CTA)
#endif
    __syncthreads();
    // the T-table image landed (the bulk copy overlapped the first prologue);
    // every later lookup of the run finds it in place
    tables_bulk_wait(&L.tbar, 0u);
#if NBA_RING_TRACE
    if (tid == 0 && R.ts) *RTR(1, 15) = gtimer();          // start-up: tables landed (row 1)
#endif
    unsigned long long c_ok = 0, c_drop = 0, c_in = 0, c_out = 0;
    for (uint32_t bi = 0; bi < n_batches; bi++) {
        const BatchArgs B = slots[(first + bi) % n_slots];
#if NBA_RING_TRACE
        if (tid == 0 && R.ts) *RTR(bi, 0) = gtimer();
#endif
        if (NBA_PIPE_PRO_DELAY && tid == 0) L.it0 = (uint32_t)gtimer();
        // lanes: the packet (known since the previous batch); its SA line and
        // round keys either before the barrier wait / scans / polls, whose
        // latency they then overlap (long or length-divergent batches, as
        // decided by the prologue warps), or after them (uniform short ones)
        const uint32_t ppc = fused_ppc(B.n, G);
        const uint32_t p_begin = cta * ppc;
        const uint32_t p_end = min(B.n, p_begin + ppc);
        const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
        uint32_t pk = 0, info = 0, sa = INVALID_SA, inoff = 0, outoff = 0;
        bool have = false;
        const bool early = NBA_PIPE_EARLY_KEYS == 1 ? true
                         : NBA_PIPE_EARLY_KEYS == 0 ? false : (L.pstat[2] & 1u) != 0u;
        const bool uniform = (L.pstat[2] & 4u) != 0u;    // the batch's packets share one length bin
        // one AES step per packet (and at most 448): producer / consumer warps
        const bool split = NBA_PIPE_SPLIT && L.pstat[1] <= 1u;
        PktPre pp = {};
        if (!isP && !split) {
            const uint32_t run = L.wrun[warp];          // LPT placement of the runs
            const uint32_t pos = 32u * run + lane;
            have = run != 0xffu && pos < cnt;
            pk = have ? L.perm[pos] : 0u;
            info = have ? L.info[pk] : 0u;
            sa = (info & INFO_OK) ? L.sa[pk] : INVALID_SA;
            inoff = have ? L.inoff[pk] : 0u;
            outoff = have ? L.outoff[pk] : 0u;
            if (NBA_RK_ASYNC && (info & INFO_OK)) {
                // round keys by cp.async and the SA line (with round keys 1, 2):
                // in flight during the barrier wait / scans / polls
                rk_async_issue(T.rk, sa, L, H, tid);
                pp = load_pkt_pre(T, B.in_buf, sa, inoff, true, 0u);
                ldg_nc_v8(&T.sal[(size_t)sa * SAL_U4 + 6], pp.r1, pp.r2);
            } else if (early && (info & INFO_OK)) {
                pp = load_pkt_pre(T, B.in_buf, sa, inoff, true, 0u);
                expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
            }
#if NBA_RING_TRACE
            if (lane == 0 && R.ts) atomicMax(RTR(bi, 6), gtimer());
#endif
        } else if (NBA_PIPE_META_PF && bi + 2 < n_batches) {
            const BatchArgs B2 = slots[(first + bi + 2) % n_slots];
            pipe_prefetch_meta(B2, fused_ppc(B2.n, G), pt);      // two batches ahead, into L2
        }
#if NBA_RING_TRACE
        pipe_sequence(T, work_of(bi), B, ppc, base0 + (bi + 1) * G, epoch_of(bi), L, RTR(bi, 0));
#else
        pipe_sequence(T, work_of(bi), B, ppc, base0 + (bi + 1) * G, epoch_of(bi), L);
#endif
        if (!isP && split) {
            const uint32_t ep = bi + 1u;                 // ready-flag value of this batch
            volatile uint32_t *ready = L.tailf;
            if (tid < SPLIT_PROD) {
                // producer: packets tid, tid + 192, tid + 384
                uint32_t f_info[3], f_sa[3], f_q[3], f_in[3];
#pragma unroll
                for (uint32_t k = 0; k < 3u; k++) {
                    const uint32_t j = tid + k * SPLIT_PROD;
                    f_info[k] = j < cnt ? L.info[j] : 0u;
                    f_sa[k] = j < cnt ? L.sa[j] : 0u;
                    f_q[k] = j < cnt ? L.seq[j] : 0u;
                    f_in[k] = j < cnt ? L.inoff[j] : 0u;
                }
                bar_arrive_n(2, F_THREADS);              // fields taken: the arrays are free
#define NBA_SEL3(a, k) ((k) == 0u ? a[0] : (k) == 1u ? a[1] : a[2])   // (no local memory)
#pragma unroll 1
                for (uint32_t k = 0; k < 3u; k++) {
                    const uint32_t j = tid + k * SPLIT_PROD;
                    const uint32_t info_k = NBA_SEL3(f_info, k), q_k = NBA_SEL3(f_q, k);
                    if (j < cnt && (info_k & INFO_OK) && q_k != 0u && !NBA_PROLOGUE_ONLY) {
                        split_produce(T, B, L, H, lane4r, tid, NBA_SEL3(f_sa, k), info_k, q_k,
                                      NBA_SEL3(f_in, k), j);
                        __threadfence_block();
                        ready[j] = ep;
                    }
                }
            } else {
                // consumer: packets u, u + 256 (u = tid - 192)
                const uint32_t u = tid - SPLIT_PROD;
                uint32_t f_info[2], f_sa[2], f_q[2], f_in[2], f_out[2];
#pragma unroll
                for (uint32_t k = 0; k < 2u; k++) {
                    const uint32_t j = u + k * SPLIT_CONS;
                    f_info[k] = j < cnt ? L.info[j] : 0u;
                    f_sa[k] = j < cnt ? L.sa[j] : 0u;
                    f_q[k] = j < cnt ? L.seq[j] : 0u;
                    f_in[k] = j < cnt ? L.inoff[j] : 0u;
                    f_out[k] = j < cnt ? L.outoff[j] : 0u;
                }
                bar_arrive_n(2, F_THREADS);
#define NBA_SEL2(a, k) ((k) == 0u ? a[0] : a[1])
#pragma unroll 1
                for (uint32_t k = 0; k < 2u; k++) {
                    const uint32_t j = u + k * SPLIT_CONS;
                    if (j >= cnt) continue;
                    const uint32_t pkt = p_begin + j;
                    const uint32_t info_k = NBA_SEL2(f_info, k), q_k = NBA_SEL2(f_q, k);
                    if ((info_k & INFO_OK) && q_k != 0u) {
                        if (!NBA_PROLOGUE_ONLY) {
                            while (ready[j] != ep) __nanosleep(32);
                            __threadfence_block();
                            split_consume(T, B, H, NBA_SEL2(f_sa, k), info_k, q_k, NBA_SEL2(f_in, k),
                                          NBA_SEL2(f_out, k), j);
                        }
                        const uint32_t Dp = info_k & 0x7ffu;
                        const uint32_t Lp = 48u + esp_C(Dp);
                        B.out_len[pkt] = (uint16_t)Lp;
                        c_ok++;
                        c_in += Dp;
                        c_out += Lp;
                    } else {
                        B.out_len[pkt] = 0;
                        c_drop++;
                    }
                }
#undef NBA_SEL2
#undef NBA_SEL3
            }
        } else if (!isP) {
            const uint32_t q32 = have ? L.seq[pk] : 0u;
            bar_arrive_n(2, F_THREADS);                  // fields taken: the arrays are free
            if (have) {
                const uint32_t pkt = p_begin + pk;
                if (NBA_RK_ASYNC && (info & INFO_OK)) rk_async_wait();   // (dropped ones too)
                if ((info & INFO_OK) && q32 != 0u) {
                    if (!NBA_RK_ASYNC && !early) {
                        pp = load_pkt_pre(T, B.in_buf, sa, inoff, true, 0u);
                        expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
                    }
#ifdef NBA_STAGGER_NS   // experiment: delay the upper lane warps (phase-locking of AES / SHA-1)
                    if (warp >= 7u) __nanosleep(NBA_STAGGER_NS);
#endif
                    uint32_t t_start = 0;
                    if (NBA_PIPE_STAGGER && uniform) {       // one-length batches only
                        t_start = (uint32_t)gtimer();
                        if (warp >= PIPE_LANE_WARPS / 2u) {   // the upper half waits
                            const uint32_t d = L.stag_ns;
                            while ((uint32_t)gtimer() - t_start < d) __nanosleep(256);
                        }
                    }
#if NBA_RING_TRACE
                    // lane timeline of the first batches (CTAs 0..3): esp_packet's clock64
                    // segments, then globaltimer at its start / end
                    unsigned long long *ldbg = (R.ts && cta < 4u && bi < 4u)
                        ? R.ts + (size_t)n_batches * G * 16u + ((size_t)(bi * 4u + cta) * PIPE_MAX_PPC + tid) * 8u
                        : nullptr;
                    if (ldbg) ldbg[6] = gtimer();
#else
                    unsigned long long *ldbg = nullptr;
#endif
                    if (!NBA_PROLOGUE_ONLY)   // (debug A/B: the ring without the lane work)
                        esp_packet(T, B, L, H, lane4r, tid, sa, info, q32, inoff, outoff, pp, ldbg,
                                   (NBA_PIPE_STAGGER && uniform && warp < PIPE_LANE_WARPS / 2u)
                                       ? &L.stag_acc : nullptr,
                                   t_start);
#if NBA_RING_TRACE
                    if (ldbg) ldbg[7] = gtimer();
#endif
                    const uint32_t Dp = info & 0x7ffu;
                    const uint32_t Lp = 48u + esp_C(Dp);
                    B.out_len[pkt] = (uint16_t)Lp;
                    c_ok++;
                    c_in += Dp;
                    c_out += Lp;
                } else {
                    B.out_len[pkt] = 0;
                    c_drop++;
                }
            }
            if (NBA_PIPE_PRO_DELAY && lane == 0) atomicMax(&L.lanes_acc, (uint32_t)gtimer() - L.it0);
#if NBA_RING_TRACE
            if (lane == 0 && R.ts) atomicMax(RTR(bi, 3), gtimer());
#endif
        } else {
            bar_sync_n(2, F_THREADS);                    // every lane took its fields
            if (NBA_PIPE_PRO_DELAY) {   // off the lanes' AES phase (its shared-memory load)
                const uint32_t t0 = (uint32_t)gtimer(), d = L.pro_delay;
                while ((uint32_t)gtimer() - t0 < d) __nanosleep(256);
            }
#ifdef NBA_PRO_DELAY_NS   // experiment: start the next batch's prologue later (after the AES phase)
            {
                const uint32_t t0 = (uint32_t)gtimer();
                while ((uint32_t)gtimer() - t0 < NBA_PRO_DELAY_NS) __nanosleep(256);
            }
#endif
            if (bi + 1 < n_batches) {
                const BatchArgs Bn = slots[(first + bi + 1) % n_slots];
                PipeMeta meta;
                pipe_load_meta(Bn, fused_ppc(Bn.n, G), pt, meta);
#if NBA_RING_TRACE
                pipe_prologue(T, work_of(bi + 1), Bn, fused_ppc(Bn.n, G), base0 + (bi + 2) * G,
                              epoch_of(bi + 1), L, pt, (bi + 1) & 1u, meta, RTR(bi, 0));
#else
                pipe_prologue(T, work_of(bi + 1), Bn, fused_ppc(Bn.n, G), base0 + (bi + 2) * G,
                              epoch_of(bi + 1), L, pt, (bi + 1) & 1u, meta);
#endif
            }
        }
        __syncthreads();                                  // batch bi done, bi + 1 prepared
        if (NBA_PIPE_STAGGER && tid == 0) {               // next batch's delay of the upper warps
            L.stag_ns = (uint32_t)(((unsigned long long)L.stag_acc * NBA_PIPE_STAGGER) >> 8);
            L.stag_acc = 0u;
        }
        if (NBA_PIPE_PRO_DELAY && tid == 0) {             // and of the prologue warps
            L.pro_delay = min(4000u, L.lanes_acc >> 2);
            L.lanes_acc = 0u;
        }
#if NBA_RING_TRACE
        if (tid == 0 && R.ts) *RTR(bi, 5) = gtimer();
#else
        if (R.ts && tid == 0) atomicMax(&R.ts[1u + bi], gtimer());
#endif
    }
    // counters (as fused_body), device state for the next launch
    if (tid < 4) L.cnt[tid] = 0ull;
    __syncthreads();
    const unsigned long long s0 = warp_sum_u64(c_ok), s1 = warp_sum_u64(c_drop);
    const unsigned long long s2 = warp_sum_u64(c_in), s3 = warp_sum_u64(c_out);
    if (lane == 0) {
        if (s0) atomicAdd(&L.cnt[0], s0);
        if (s1) atomicAdd(&L.cnt[1], s1);
        if (s2) atomicAdd(&L.cnt[2], s2);
        if (s3) atomicAdd(&L.cnt[3], s3);
    }
    __syncthreads();
    if (tid < 4 && L.cnt[tid]) atomicAdd(&W.counters[tid], L.cnt[tid]);
    if (tid == 4 && cta == 0) {
        atomicAdd(&W.counters[4], (unsigned long long)n_batches);
        W.ctl[CTL_BAR_BASE] = base0 + n_batches * G;   // one barrier per batch
        W.ctl[CTL_EPOCH] = epoch_of(n_batches - 1u);      // the last batch's epoch
    }
}

// ----------------------------------------------- free-running lane warps
// k_fused_ring_free: the pipelined ring without the end-of-batch CTA barrier,
// for batches of mixed lengths, where one warp's run of long packets sets
// the batch time while the others wait (profiles/r02be_imix_balance.md).
// The two side warps run, per batch j: wait until every lane warp took its
// fields of batch j - 1 (smem counter fr_taken), the prologue of batch j
// (metadata, ranks, counts, arrival at its grid barrier), the run placement
// (the batch's runs, longest first, onto the lane warps with the least
// cumulative assigned cost: a long run goes to a warp that will be free
// early), the grid barrier, this CTA's share of the row scans and the polls
// of its packets' bases (the sequence numbers), then publish batch j (smem
// flag fr_ready).  A lane warp, per batch: wait for fr_ready, take its run's
// fields, count itself in fr_taken, encrypt its packets -- so a warp that
// finished a short run starts the next batch while a long run is still
// going.  Same results as k_fused_ring_pipe (the sequence numbers are the
// per-SA order of the batch, not the order of completion).
// Measured (profiles/ab/r02bh_forms.txt, the trace in DESIGN.md §9): SLOWER
// than k_fused_ring_pipe at every size (64 B 42.1 vs 22.2 us, IMIX 169 vs 88):
// the side warps' chain per batch (prologue ~32 us under the lanes' load,
// grid barrier behind the slowest CTA, row scans and polls by two warps
// ~12 us) becomes the period.  Opt-in only (nba_ipsec_ring_set_form FREE).
constexpr uint32_t FR_SPIN_MAX = 1u << 26;    // bounded waits: a kernel error, never a hang

__device__ __forceinline__ void fr_wait_ge(const uint32_t *p, uint32_t v)
{
    for (uint32_t k = 0; *reinterpret_cast<const volatile uint32_t *>(p) < v; k++) {
        if (k > FR_SPIN_MAX) __trap();
        __nanosleep(64);
    }
    __threadfence_block();
}

// The batch's grid barrier wait, this CTA's share of the row scans, and the
// polls of its packets' published bases, by the 64 side threads: L.seq[j]
// turns from the CTA rank into the ESP sequence number (0: dropped).
__device__ __forceinline__ void fr_side_sequence(const DevTable &T, const DevWork &W, uint32_t cnt,
                                                 uint32_t bar_target, uint32_t epoch, FusedLo &L,
                                                 uint32_t pt)
{
    const uint32_t G = gridDim.x, cta = blockIdx.x, lane = pt & 31u, pw = pt >> 5;
    if (pt == 0) {
        uint32_t v;
        for (uint32_t k = 0;; k++) {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&W.ctl[CTL_BAR_MONO]) : "memory");
            if ((int)(v - bar_target) >= 0) break;
            if (k > FR_SPIN_MAX) __trap();
            __nanosleep(64);
        }
    }
    bar_sync_n(1, PIPE_P);
    pipe_scan_rows(T, W, cta * 2u + pw, G * 2u, G, lane, epoch);
    unsigned long long v[PR];
    uint32_t sa_r[PR];
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {
        const uint32_t j = r * PIPE_P + pt;
        const bool ok = j < cnt && (L.info[j] & INFO_OK);
        sa_r[r] = ok ? L.sa[j] : INVALID_SA;
        v[r] = ok ? ld_relaxed_u64(&W.hbase[(size_t)sa_r[r] * G + cta]) : 0ull;
    }
#pragma unroll
    for (uint32_t r = 0; r < PR; r++) {
        const uint32_t j = r * PIPE_P + pt;
        if (j >= cnt) continue;
        uint32_t q32 = 0;
        if (sa_r[r] != INVALID_SA) {
            const unsigned long long *pb = &W.hbase[(size_t)sa_r[r] * G + cta];
            for (uint32_t k = 0; (uint32_t)(v[r] >> 33) != epoch; k++) {
                if (k > FR_SPIN_MAX) __trap();
                v[r] = ld_relaxed_u64(pb);
            }
            const unsigned long long q = (v[r] & ((1ull << 33) - 1ull)) + 1ull + L.seq[j];
            q32 = q <= 0xffffffffull ? (uint32_t)q : 0u;   // RFC 4303 §3.3.3: never cycle
        }
        L.seq[j] = q32;
    }
    bar_sync_n(1, PIPE_P);
}

// Run placement by cumulative cost (side warp 0): the lane warp with the
// k-th smallest cumulative cost takes the run with the k-th largest cost
// (run r = sorted positions 32 r ..; cost as the LPT placement's).
__device__ __forceinline__ void fr_place(FusedLo &L, uint32_t cnt, uint32_t lane)
{
    const uint32_t nruns = (cnt + 31u) / 32u;
    uint32_t cost = 0;
    if (lane < nruns) {
        const uint32_t info = L.info[L.perm[32u * lane]];
        const uint32_t C = esp_C(info & 0x7ffu);
        cost = (info & INFO_OK) ? 8u * (esp_nsha_inner(C) + 1u) + 3u * ((C + 15u) >> 4) : 1u;
    }
    uint32_t crank = 0;                            // runs costlier than this one (ties by index)
#pragma unroll
    for (uint32_t o = 0; o < PIPE_LANE_WARPS; o++) {
        const uint32_t co = __shfl_sync(0xffffffffu, cost, o);
        crank += (o < nruns && (co > cost || (co == cost && o < lane))) ? 1u : 0u;
    }
    const uint32_t w = lane;                       // lane w speaks for lane warp w
    const uint32_t ld = w < PIPE_LANE_WARPS ? L.fr_load[w] : 0xffffffffu;
    uint32_t rank = 0;                             // among the 14 warps, ties by index
#pragma unroll
    for (uint32_t o = 0; o < PIPE_LANE_WARPS; o++) {
        const uint32_t lo = __shfl_sync(0xffffffffu, ld, o);
        rank += (lo < ld || (lo == ld && o < w)) ? 1u : 0u;
    }
    uint32_t run = 0xffu, c_r = 0;                 // the run of cost rank `rank`
#pragma unroll
    for (uint32_t o = 0; o < PIPE_LANE_WARPS; o++) {
        const uint32_t cr = __shfl_sync(0xffffffffu, crank, o);
        const uint32_t co = __shfl_sync(0xffffffffu, cost, o);
        if (o < nruns && cr == rank) {
            run = o;
            c_r = co;
        }
    }
    if (w < PIPE_LANE_WARPS) {
        L.wrun[w] = (uint8_t)run;
        L.fr_load[w] = ld + c_r;
    }
    // keep the loads small: subtract the minimum
    const uint32_t nl = w < PIPE_LANE_WARPS ? L.fr_load[w] : 0xffffffffu;
    const uint32_t mn = __reduce_min_sync(0xffffffffu, nl);
    if (w < PIPE_LANE_WARPS) L.fr_load[w] = nl - mn;
}

__global__ void __launch_bounds__(F_THREADS, 1)
k_fused_ring_free(DevTable T, DevWork W, const BatchArgs *slots, RingRun R, uint16_t *hist_b)
{
    const uint32_t n_slots = R.n_slots, n_batches = R.n_batches, first = R.first;
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, cta = blockIdx.x;
    if (n_batches == 0) return;
    if (!NBA_RING_TRACE && R.ts && cta == 0 && tid == 0) R.ts[0] = gtimer();
    const uint32_t base0 = *reinterpret_cast<volatile uint32_t *>(&W.ctl[CTL_BAR_BASE]);
    const uint32_t ep0 = *reinterpret_cast<volatile uint32_t *>(&W.ctl[CTL_EPOCH]);
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
    tables_stage(tabs, T, &L.tbar, true);   // bulk copy, waited for before the first lookup
    if (tid < NBINS) L.bins[tid] = 0u;
    if (tid < 16) L.fr_load[tid] = 0u;
    if (tid == 0) {
        L.fr_ready = 0u;
        L.fr_taken = 0u;
    }
    for (uint32_t k = tid; k < 2u * F_SUPER; k += F_THREADS) {
        L.hkey[k] = INVALID_SA;
        L.hmask[k] = 0u;
        (&L.aux0[0])[k] = 0u;                     // the prologue's second count array
    }
    __syncthreads();
    auto epoch_of = [&](uint32_t bi) { return ((ep0 + bi) % 0x7fffffffu) + 1u; };
    auto work_of = [&](uint32_t bi) {
        DevWork Wb = W;
        if (bi & 1u) Wb.hist16 = hist_b;
        return Wb;
    };
    unsigned long long c_ok = 0, c_drop = 0, c_in = 0, c_out = 0;
    if (tid >= PIPE_MAX_PPC) {
        // ---- side warps: prepare every batch of the run in order
        const uint32_t pt = tid - PIPE_MAX_PPC;
        for (uint32_t bi = 0; bi < n_batches; bi++) {
            const BatchArgs B = slots[(first + bi) % n_slots];
            const uint32_t ppc = fused_ppc(B.n, G);
            const uint32_t p_begin = cta * ppc;
            const uint32_t p_end = min(B.n, p_begin + ppc);
            const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
            if (bi > 0) {                          // the arrays are free: batch bi - 1 taken
                if (pt == 0) fr_wait_ge(&L.fr_taken, PIPE_LANE_WARPS * bi);
                bar_sync_n(1, PIPE_P);
            }
#if NBA_RING_TRACE
            if (pt == 0 && R.ts) *RTR(bi, 0) = gtimer();
#endif
            PipeMeta meta;
            pipe_load_meta(B, ppc, pt, meta);
            if (bi + 1 < n_batches) {
                const BatchArgs B1 = slots[(first + bi + 1) % n_slots];
                pipe_prefetch_meta(B1, fused_ppc(B1.n, G), pt);
            }
            pipe_prologue(T, work_of(bi), B, ppc, base0 + (bi + 1) * G, epoch_of(bi), L, pt, bi & 1u, meta);
            if (pt < 32u) fr_place(L, cnt, pt);
#if NBA_RING_TRACE
            if (pt == 0 && R.ts) *RTR(bi, 1) = gtimer();
#endif
            fr_side_sequence(T, work_of(bi), cnt, base0 + (bi + 1) * G, epoch_of(bi), L, pt);
            if (pt == 0) {
                __threadfence_block();
                *reinterpret_cast<volatile uint32_t *>(&L.fr_ready) = bi + 1u;
            }
#if NBA_RING_TRACE
            if (pt == 0 && R.ts) *RTR(bi, 2) = gtimer();
#endif
        }
    } else {
        // ---- lane warps: each batch as soon as it is prepared
        tables_bulk_wait(&L.tbar, 0u);
        for (uint32_t bi = 0; bi < n_batches; bi++) {
            const BatchArgs B = slots[(first + bi) % n_slots];
            const uint32_t ppc = fused_ppc(B.n, G);
            const uint32_t p_begin = cta * ppc;
            const uint32_t p_end = min(B.n, p_begin + ppc);
            const uint32_t cnt = p_end > p_begin ? p_end - p_begin : 0u;
#if NBA_RING_TRACE
            const unsigned long long t_w = gtimer();
#endif
            if (lane == 0) fr_wait_ge(&L.fr_ready, bi + 1u);
            __syncwarp();
            __threadfence_block();
#if NBA_RING_TRACE
            if (lane == 0 && R.ts) {
                atomicMax(RTR(bi, 3), gtimer());          // the latest take
                atomicMax(RTR(bi, 6), gtimer() - t_w);    // the longest wait for the batch
            }
#endif
            const uint32_t run = L.wrun[warp];
            const uint32_t pos = 32u * run + lane;
            const bool have = run != 0xffu && pos < cnt;
            const uint32_t pk = have ? L.perm[pos] : 0u;
            const uint32_t info = have ? L.info[pk] : 0u;
            const uint32_t sa = (info & INFO_OK) ? L.sa[pk] : INVALID_SA;
            const uint32_t inoff = have ? L.inoff[pk] : 0u;
            const uint32_t outoff = have ? L.outoff[pk] : 0u;
            const uint32_t q32 = have ? L.seq[pk] : 0u;
            __syncwarp();
            if (lane == 0) {                       // fields taken: the side may reuse the arrays
                __threadfence_block();
                atomicAdd(&L.fr_taken, 1u);
            }
            if (have) {
                const uint32_t pkt = p_begin + pk;
                if ((info & INFO_OK) && q32 != 0u) {
                    PktPre pp = load_pkt_pre(T, B.in_buf, sa, inoff, true, 0u);
                    expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
                    esp_packet(T, B, L, H, lane4r, tid, sa, info, q32, inoff, outoff, pp, nullptr);
                    const uint32_t Dp = info & 0x7ffu;
                    const uint32_t Lp = 48u + esp_C(Dp);
                    B.out_len[pkt] = (uint16_t)Lp;
                    c_ok++;
                    c_in += Dp;
                    c_out += Lp;
                } else {
                    B.out_len[pkt] = 0;
                    c_drop++;
                }
            }
#if NBA_RING_TRACE
            if (R.ts && lane == 0) atomicMax(RTR(bi, 4), gtimer());   // the latest lane finish
#else
            if (R.ts && lane == 0) atomicMax(&R.ts[1u + bi], gtimer());
#endif
        }
    }
    // counters (as fused_body), device state for the next launch
    __syncthreads();
    if (tid < 4) L.cnt[tid] = 0ull;
    __syncthreads();
    const unsigned long long s0 = warp_sum_u64(c_ok), s1 = warp_sum_u64(c_drop);
    const unsigned long long s2 = warp_sum_u64(c_in), s3 = warp_sum_u64(c_out);
    if (lane == 0) {
        if (s0) atomicAdd(&L.cnt[0], s0);
        if (s1) atomicAdd(&L.cnt[1], s1);
        if (s2) atomicAdd(&L.cnt[2], s2);
        if (s3) atomicAdd(&L.cnt[3], s3);
    }
    __syncthreads();
    if (tid < 4 && L.cnt[tid]) atomicAdd(&W.counters[tid], L.cnt[tid]);
    if (tid == 4 && cta == 0) {
        atomicAdd(&W.counters[4], (unsigned long long)n_batches);
        W.ctl[CTL_BAR_BASE] = base0 + n_batches * G;   // one barrier per batch
        W.ctl[CTL_EPOCH] = epoch_of(n_batches - 1u);      // the last batch's epoch
    }
}

// ------------------------------------- role-split ring (SM specialisation)
// k_fused_ring_roles: the batch ring with CTA roles instead of warp roles.
// CTAs 0..P-1 ("sequencers") run every batch's prologue: validity (A15), the
// stable rank of each valid packet among the batch's earlier valid packets of
// its SA (index order over the whole batch), its sequence number q = seq + 1
// + rank (RFC 4303 §3.3.3: dropped once q would pass 2^32 - 1, as the oracle's
// step 2), and one 4-byte record per packet (q, 0 = drop) into a ring of
// ROLES_NREC record buffers.  CTAs P..G-1
// ("lanes", 16 warps) take batch b's records as soon as its sequencers
// published them and encrypt their packets with the same esp_packet as every
// other path.  Nothing synchronises the lane CTAs between two batches: a lane
// warp that finished batch b starts batch b + 1 once its records are there, so
// the shared-memory-bound AES and the ALU-bound SHA-1 of different warps drift
// apart instead of running in lock step (the pipelined ring's lanes spend
// most of a 64-B batch with every warp in the same phase), and the
// per-batch critical section (grid barrier, row scans, polls) leaves the lane
// SMs altogether.  Packet i of a batch always goes to the same lane (lane CTA
// i / ppc, position j = i mod ppc -> warp j mod 16, lane j / 16, so every warp
// carries ~ppc / 16 packets), so the uses of one ring slot write its output
// slots in program order.  Records are stored by packet index (coalesced
// sequencer stores; a lane's one 4-byte load per batch is scattered); a lane
// reads its packet's SA, length and offsets from the batch itself one batch
// ahead, so its SA line and round keys are ready before the record is read,
// and prefetches its next payload line into L2.  The lanes' waits and counts
// use no acquire / release fences (roles_lane_wait / roles_lane_consumed).
// Mixed-length rings of more than ROLES_NREC slots take the sorted mode (per
// batch length-sorted runs placed on the lane warps by cumulative cost,
// roles_sort_slots / roles_lanes_sorted); in the fixed-slot mode a launch's
// first batch is numbered by every CTA (roles_boot0) and the sequencers start
// at batch 1.
//
// Hand-offs (counters monotonic within a launch, zeroed by the last CTA to
// leave; s = b mod ROLES_NREC, k = b / ROLES_NREC):
//   ready[s]    += 1 per sequencer once batch b's records are written: the
//                  lanes wait for (k + 1) P (the bootstrap counts batch 0 as P);
//   consumed[s] += 1 per lane warp once it loaded its records of batch b: a
//                  sequencer starts batch b only when it reads k * (lane warps);
//   pbar        += 1 per sequencer and batch once its per-SA totals are out;
//   boot bar / done: the bootstrap's two grid barriers and its completion count.
__device__ __forceinline__ uint32_t roles_ld_acq(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void roles_red_rel(uint32_t *p, uint32_t v)
{
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ uint32_t roles_ld_relaxed(const uint32_t *p);

// Wait until *p >= target (wrapping compare) with acquire semantics: relaxed
// polls (an acquire load invalidates the SM's L1 on every iteration), then one
// acquire load of the count that satisfied it.
__device__ __forceinline__ void roles_wait_geq(const uint32_t *p, uint32_t target)
{
    while ((int32_t)(roles_ld_relaxed(p) - target) < 0) __nanosleep(32);
    (void)roles_ld_acq(p);
}

// The lanes' side of the hand-offs, without the acquire / release fences:
// an acquire load invalidates the SM's L1 (CCTL.IVALL) and a release RMW waits
// for every store the warp has in flight (MEMBAR + ERRBAR) -- together ~8% of
// the lane warps' stall samples (ncu, 64 B).  Instead: lane 0 polls with a
// relaxed load and the warp reads its records with L2 loads (ld.cg) issued
// only after the poll returned (control dependency, in-order issue; L2 is the
// point of coherence, and the sequencer's release made its records visible
// there before its count); the "consumed" count is a relaxed add whose operand
// depends, through a warp vote, on every lane's loaded record -- it cannot be
// performed before those loads returned.
__device__ __forceinline__ uint32_t roles_ld_relaxed(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void roles_lane_wait(const uint32_t *p, uint32_t target)
{
    if ((threadIdx.x & 31u) == 0)
        while ((int32_t)(roles_ld_relaxed(p) - target) < 0) __nanosleep(32);
    __syncwarp();
}

__device__ __forceinline__ void roles_lane_consumed(uint32_t *p, uint32_t q)
{
    uint32_t z;
    asm("and.b32 %0, %1, 0;" : "=r"(z) : "r"(q));     // 0, opaque: depends on the load of q
    z = __ballot_sync(0xffffffffu, z != 0u);          // every lane's record has returned
    if ((threadIdx.x & 31u) == 0)
        asm volatile("red.relaxed.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(1u + z) : "memory");
}

#ifndef NBA_ROLES_TRACE       // debug variant: sequencer 0's phase stamps per batch and lane CTA 0's
#define NBA_ROLES_TRACE 0     //   record arrival, after ts[0..n_batches] (tools/roles_trace.py)
#endif
#if NBA_ROLES_TRACE
#define RLT(bi, k) (R.ts + 1u + R.n_batches + (size_t)(bi) * 8u + (k))
#endif
#ifndef NBA_ROLES_WARM        // experiment: lanes' warm-up pass (0 off, 1 all warps, 2 warp 0, 3 warps 0-3)
#define NBA_ROLES_WARM 0
#endif
#ifndef NBA_ROLES_WARM_D      // experiment: the warm-up packet's length (0: the lane's own, up to 114)
#define NBA_ROLES_WARM_D 0
#endif
#ifndef NBA_ROLES_SAL_AHEAD   // lanes: the next packet's SA line loaded at the end of an iteration
#define NBA_ROLES_SAL_AHEAD 0       // (measured: 64 B 20.5 -> 20.7 us, 128 B 29.3 -> 28.4, 512 B 73.6 -> 74.6, 1024 B 134 -> 137)
#endif
#ifndef NBA_ROLES_SAL_L1      // lanes: L1 prefetch of the next packet's SA line after each packet
#define NBA_ROLES_SAL_L1 0
#endif
#ifndef NBA_ROLES_RK_ASYNC    // lanes: round keys 3..10 by cp.async from the SA's schedule instead of
#define NBA_ROLES_RK_ASYNC 0  //   expanded from the key (1)
#endif
#ifndef NBA_ROLES_MATCH       // sequencer: equal-SA groups by MATCH.ANY (1) or 12 ballots (0)
#define NBA_ROLES_MATCH 0
#endif
#ifndef NBA_ROLES_AG          // sequencer: rounds of 32 packets whose metadata loads are in flight together
#define NBA_ROLES_AG 8
#endif

// Batch-0 bootstrap (fixed-slot mode): the sequencers would need ~20 us for a
// launch's first batch (their ranking is compute-bound and nothing overlaps
// it), so every CTA numbers batch 0 instead, the pipelined ring's way: CTA c
// takes packets [c ppc0, (c + 1) ppc0) (one per thread), ranks them per SA
// (12-ballot groups in each warp, the warps' group sizes in rows in global
// memory, so the lane CTAs' shared memory -- T-tables in flight, slot table --
// is untouched), writes each packet's rank to rank0 and its per-SA counts into
// column c of hist0 (zeroed by CTA c first); after a grid barrier each warp
// turns one SA row into exclusive prefixes over the CTAs in place (and the row
// total into tot0); after a second barrier batch 0's numbers are known: a lane
// computes its packet's q = SA counter + 1 + hist0[sa][i / ppc0] + rank0[i]
// (saturating as the sequencers) without a record, and the last CTA through
// counts batch 0 as published for the sequencers' bookkeeping (ready[0] += P,
// pbar += P).
__device__ __forceinline__ uint32_t roles_boot0(const DevTable &T, const BatchArgs *slots, const RingRun &R,
                                                const RolesBufs &Q, uint32_t sa_mine)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t G = gridDim.x, c = blockIdx.x, n_sa = T.n_sa;
    const BatchArgs B = slots[R.first % R.n_slots];
    const uint32_t n = B.n, ppc0 = (n + G - 1u) / G, i = c * ppc0 + tid;
    const bool in = tid < ppc0 && i < n;
    const uint32_t s = in ? B.sa_idx[i] : INVALID_SA, D = in ? (uint32_t)B.in_len[i] : 0u;
    const bool cand = in && s < n_sa && D >= MIN_D && D <= MAX_D;
    uint16_t *rows = Q.rows0 + (size_t)c * 16u * n_sa;                   // [16][n_sa]
    uint32_t *bar = Q.ctl + 2u * ROLES_NREC + 2u, *done = bar + 1;
#if NBA_ROLES_TRACE
    if (R.ts && tid == 0) atomicMax(RLT(1, 6), gtimer());   // the latest boot start
#endif
#if NBA_ROLES_TRACE
    if (R.ts && c == 0 && tid == 0) *RLT(0, 0) = gtimer();
#endif
    for (uint32_t k = tid; k < 2u * n_sa; k += F_THREADS)               // 16 x n_sa u16 = 2 n_sa uint4
        reinterpret_cast<uint4 *>(rows)[k] = make_uint4(0u, 0u, 0u, 0u);
    for (uint32_t sa = tid; sa < n_sa; sa += F_THREADS) Q.hist0[(size_t)sa * G + c] = 0u;
    __syncthreads();
#if NBA_ROLES_TRACE
    if (R.ts && c == 0 && tid == 0) *RLT(0, 1) = gtimer();
#endif
    const uint32_t key = cand ? s : 0x800u;
    uint32_t peers = 0xffffffffu;
#pragma unroll
    for (uint32_t bit = 0; bit < 12u; bit++) {
        const bool on = (key >> bit) & 1u;
        const uint32_t m = __ballot_sync(0xffffffffu, on);
        peers &= on ? m : ~m;
    }
    const uint32_t leader = (uint32_t)__ffs(peers) - 1u;
    if (cand && lane == leader) rows[warp * n_sa + s] = (uint16_t)__popc(peers);
    __syncthreads();
    uint32_t pre = 0u, tot = 0u;
    bool first = true;                                   // the lowest warp holding the SA
    if (cand)
        for (uint32_t w = 0; w < 16u; w++) {
            const uint32_t v = __ldcg(&rows[w * n_sa + s]);
            if (w < warp) {
                pre += v;
                first = first && v == 0u;
            }
            tot += v;
        }
    if (in) Q.rank0[i] = (uint16_t)(pre + __popc(peers & lanemask_lt()));
    if (cand && lane == leader && first) Q.hist0[(size_t)s * G + c] = tot;
    __syncthreads();
#if NBA_ROLES_TRACE
    if (R.ts && c == 0 && tid == 0) *RLT(0, 2) = gtimer();
#endif
    if (tid == 0) {
#if NBA_ROLES_TRACE
        if (R.ts) atomicMax(RLT(0, 6), gtimer());       // the latest arrival (any CTA)
#endif
        __threadfence();
        roles_red_rel(bar, 1u);
        roles_wait_geq(bar, G);
    }
    __syncthreads();
#if NBA_ROLES_TRACE
    if (R.ts && c == 0 && tid == 0) *RLT(0, 3) = gtimer();
#endif
    // exclusive prefixes over the CTAs, one warp per SA row (lane l: columns [5l, 5l + 5))
    for (uint32_t sa = c + warp * G; sa < n_sa; sa += 16u * G) {
        uint32_t v[5], sum = 0;
#pragma unroll
        for (uint32_t k = 0; k < 5u; k++) {
            const uint32_t col = 5u * lane + k;
            v[k] = col < G ? __ldcg(&Q.hist0[(size_t)sa * G + col]) : 0u;
            sum += v[k];
        }
        uint32_t x = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= (uint32_t)o) x += y;
        }
        uint32_t run = x - sum;
#pragma unroll
        for (uint32_t k = 0; k < 5u; k++) {
            const uint32_t col = 5u * lane + k;
            if (col < G) Q.hist0[(size_t)sa * G + col] = run;
            run += v[k];
        }
        if (lane == 31u) Q.tot0[sa] = x;
    }
    const uint32_t seq_mine = sa_mine < n_sa ? __ldcg(&T.seq[sa_mine]) : 0u;   // (before barrier 2)
    __syncthreads();
#if NBA_ROLES_TRACE
    if (R.ts && c == 0 && tid == 0) *RLT(0, 4) = gtimer();
#endif
    if (tid == 0) {
#if NBA_ROLES_TRACE
        if (R.ts) atomicMax(RLT(0, 7), gtimer());
#endif
        __threadfence();
        roles_red_rel(bar, 1u);
        roles_wait_geq(bar, 2u * G);
        if (atomicAdd(done, 1u) == G - 1u) {
            roles_red_rel(Q.ctl, Q.npro);                              // ready[0]
            roles_red_rel(Q.ctl + 2u * ROLES_NREC, Q.npro);            // pbar: batch 0's arrivals
        }
    }
    __syncthreads();
#if NBA_ROLES_TRACE
    if (R.ts && c == 0 && tid == 0) *RLT(0, 5) = gtimer();
#endif
    return seq_mine;
}

// A lane's batch-0 sequence number after the bootstrap (0 = drop); seq0 = the
// SA's counter, read before the bootstrap's barriers.
__device__ __forceinline__ uint32_t roles_boot_q(const RolesBufs &Q, const BatchArgs &B, uint32_t i,
                                                 uint32_t sa, uint32_t seq0)
{
    const uint32_t G = gridDim.x, ppc0 = (B.n + G - 1u) / G;
    const unsigned long long q64 = (unsigned long long)seq0 + __ldcg(&Q.hist0[(size_t)sa * G + i / ppc0]) +
                                   __ldcg(&Q.rank0[i]) + 1ull;
    return q64 <= 0xffffffffull ? (uint32_t)q64 : 0u;
}

// Sorted mode (mixed-length rings), per lane CTA of this sequencer, one warp
// each: the CTA's packets in a stable counting sort by HMAC length bin
// (longest first, invalid last), cut into runs of 32 sorted positions; run r
// goes to the lane warp with the least work assigned so far (LPT over the
// warps' cumulative cost, Q.cum, so the long runs rotate among the warps from
// batch to batch); d16[packet] becomes the packet's lane slot (warp * 32 +
// position in the run).  Slots left without a packet get the record
// {0, 0xffffffff}.  A run's cost: 8 (SHA-1 blocks + 1) + 3 AES steps of its
// first (longest) packet, ~11 x inner SHA-1 blocks + 8.
__device__ __noinline__ void roles_sort_slots(uint4 *rec, uint32_t *cumb, uint16_t *d16, const uint32_t *sav,
                                              uint32_t (*hw)[NBINS], uint32_t r0, uint32_t n,
                                              uint32_t ppc, uint32_t cbeg, uint32_t cend)
{
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    for (uint32_t cc = cbeg + warp; cc < cend; cc += 16u) {
        const uint32_t pb = min(n, cc * ppc), pe = min(n, pb + ppc), cnt = pe - pb;
        auto bin_of = [&](uint32_t i) {
            const bool ok = sav[i - r0] != 0xffffffffu;
            return hmac_bin(ok, esp_C(d16[i - r0]));
        };
        hw[warp][lane] = 0u;
        __syncwarp();
        for (uint32_t g = pb; g < pe; g += 32u)
            warp_agg_add(hw[warp], g + lane < pe ? bin_of(g + lane) : 0u, g + lane < pe);
        __syncwarp();
        const uint32_t cb = hw[warp][lane];           // lane = bin: count, exclusive prefix
        uint32_t x = cb;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= (uint32_t)o) x += y;
        }
        const uint32_t base = x - cb;
        hw[warp][lane] = base;
        // runs: the bin of each run's first position, its cost; LPT onto the warps
        const uint32_t nruns = (cnt + 31u) / 32u;
        uint32_t binr = NBINS - 1u;
        for (uint32_t b = 0; b < (uint32_t)NBINS; b++) {
            const uint32_t bb = __shfl_sync(0xffffffffu, base, b), cbb = __shfl_sync(0xffffffffu, cb, b);
            if (cbb > 0u && bb <= 32u * lane) binr = b;      // the last such bin holds position 32 lane
        }
        const uint32_t cost = binr == NBINS - 1u ? 1u : 11u * (NBINS - 1u - binr) + 8u;
        uint32_t cum = lane < 16u ? cumb[cc * 16u + lane] : 0xffffffffu;
        uint32_t wsl = 0xffu;                          // lane r: warp of run r
        bool taken = lane >= 16u;                      // lane w: warp w holds a run of this batch
        for (uint32_t r = 0; r < nruns; r++) {         // (nruns <= 16: one run per warp)
            const uint32_t cr = __shfl_sync(0xffffffffu, cost, r);
            const uint32_t v = __reduce_min_sync(0xffffffffu, taken ? 0xffffffffu
                                                                    : (min(cum, 0x7ffffffu) << 5) | lane);
            const uint32_t w = v & 31u;
            if (lane == w) {
                cum += cr;
                taken = true;
            }
            if (lane == r) wsl = w;
        }
        const uint32_t m = __reduce_min_sync(0xffffffffu, lane < 16u ? cum : 0xffffffffu);
        if (lane < 16u) cumb[cc * 16u + lane] = cum - m;   // (kept small)
        // the run each warp holds (lane w: run or 0xffffffff)
        uint32_t myrun = 0xffffffffu;
        for (uint32_t r = 0; r < nruns; r++)
            if (__shfl_sync(0xffffffffu, wsl, r) == lane) myrun = r;
        __syncwarp();
        // stable scatter: position = bin base + rank among the earlier packets of its bin
        for (uint32_t g = pb; g < pe; g += 32u) {
            const uint32_t i = g + lane;
            const bool in = i < pe;
            const uint32_t pos = warp_agg_add(hw[warp], in ? bin_of(i) : 0u, in);
            const uint32_t w = __shfl_sync(0xffffffffu, wsl, in ? (pos >> 5) : 0u);
            if (in) d16[i - r0] = (uint16_t)(w * 32u + (pos & 31u));
        }
        // slots without a packet
        for (uint32_t sl = lane; sl < 512u; sl += 32u) {
            const uint32_t r = __shfl_sync(0xffffffffu, myrun, sl >> 5);
            if (r == 0xffffffffu || 32u * r + (sl & 31u) >= cnt)
                rec[(size_t)cc * 512u + sl] = make_uint4(0u, 0xffffffffu, 0u, 0u);
        }
        __syncwarp();
    }
}

__device__ __forceinline__ void roles_sequencer(const DevTable &T, const BatchArgs *slots, const RingRun &R,
                                                const RolesBufs &Q, uint8_t *smem, uint32_t p)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t P = Q.npro, Lc = gridDim.x - P, LW = Lc * 16u, n_sa = T.n_sa;
    // shared memory: this sequencer's range of SA indices and lengths (staged by
    // bulk copies from the batch; the SA index becomes 0xffffffff for a dropped
    // packet, the length the lane slot in sorted mode), each packet's rank,
    // per-warp SA counters, the SAs' counters and bases
    uint16_t *rank = reinterpret_cast<uint16_t *>(smem);                          // [RPP_MAX]
    uint32_t *raw_sa = reinterpret_cast<uint32_t *>(rank + ROLES_RPP_MAX);        // [RPP_MAX + 8]
    uint16_t *raw_len = reinterpret_cast<uint16_t *>(raw_sa + ROLES_RPP_MAX + 8u); // [RPP_MAX + 16]
    uint16_t *cnt = raw_len + ROLES_RPP_MAX + 16u;                                // [16][ROLES_MAX_SA]
    uint32_t *seqs = reinterpret_cast<uint32_t *>(cnt + 16u * ROLES_MAX_SA);      // [ROLES_MAX_SA]
    unsigned long long *start = reinterpret_cast<unsigned long long *>(seqs + ROLES_MAX_SA);
    uint32_t (*sorth)[NBINS] = reinterpret_cast<uint32_t (*)[NBINS]>(start + ROLES_MAX_SA);   // [16][NBINS]
    unsigned long long *mbar = reinterpret_cast<unsigned long long *>(&sorth[16][0]);
    static_assert(ROLES_RPP_MAX % 8u == 0u, "16-B aligned stash arrays");
    static_assert(ROLES_RPP_MAX * 2u + (ROLES_RPP_MAX + 8u) * 4u + (ROLES_RPP_MAX + 16u) * 2u +
                      16u * ROLES_MAX_SA * 2u + ROLES_MAX_SA * 12u + 16u * NBINS * 4u + 8u <= F_SMEM,
                  "sequencer shared memory");
    uint32_t *ready = Q.ctl, *consumed = Q.ctl + ROLES_NREC, *pbar = Q.ctl + 2u * ROLES_NREC;
    uint16_t *mycnt = cnt + warp * ROLES_MAX_SA;
    if (Q.boot) roles_boot0(T, slots, R, Q, INVALID_SA);
    for (uint32_t s = tid; s < n_sa; s += F_THREADS)
        seqs[s] = Q.boot ? (uint32_t)min((unsigned long long)__ldcg(&T.seq[s]) + __ldcg(&Q.tot0[s]), 0xffffffffull)
                         : __ldcg(&T.seq[s]);
    for (uint32_t s = lane; s < n_sa; s += 32u) mycnt[s] = 0;
    if (tid == 0) tbar_init(mbar);
    __syncthreads();
    // this sequencer's lane CTAs [cbeg, cend): its packet range is theirs
    const uint32_t cbeg = p * Lc / P, cend = (p + 1u) * Lc / P;
    for (uint32_t bi = Q.boot ? 1u : 0u; bi < R.n_batches; bi++) {
        const BatchArgs B = slots[(R.first + bi) % R.n_slots];
        const uint32_t n = B.n, ppc = (n + Lc - 1u) / Lc;
        const uint32_t r0 = min(n, cbeg * ppc), r1 = min(n, cend * ppc), rpp = r1 - r0;
        const uint32_t spw = (((rpp + 15u) / 16u) + 31u) & ~31u;   // whole rounds per warp
        const uint32_t w0 = min(r1, r0 + warp * spw), w1 = min(r1, w0 + spw);
        // the next batch's metadata lines into L2 (ahead of its phase A; batch 0's
        // at the start)
        for (uint32_t nb = bi == (Q.boot ? 1u : 0u) ? bi : bi + 1u; nb <= bi + 1u && nb < R.n_batches; nb++) {
            const BatchArgs Bn = slots[(R.first + nb) % R.n_slots];
            const uint32_t pn = (Bn.n + Lc - 1u) / Lc, a0 = min(Bn.n, cbeg * pn), a1 = min(Bn.n, cend * pn);
            const uint32_t l16 = a1 > a0 ? (2u * (a1 - a0) + 127u) / 128u + 1u : 0u;
            const uint32_t l32 = a1 > a0 ? (4u * (a1 - a0) + 127u) / 128u + 1u : 0u;
            for (uint32_t k = tid; k < l16 + l32; k += F_THREADS) {   // in_len, sa_idx
                const uint8_t *a, *e;
                if (k < l16) {
                    a = reinterpret_cast<const uint8_t *>(Bn.in_len + a0) + 128u * k;
                    e = reinterpret_cast<const uint8_t *>(Bn.in_len + a1);
                } else {
                    a = reinterpret_cast<const uint8_t *>(Bn.sa_idx + a0) + 128u * (k - l16);
                    e = reinterpret_cast<const uint8_t *>(Bn.sa_idx + a1);
                }
                if (a < e) prefetch_l2(a);
            }
        }
#if NBA_ROLES_TRACE
        if (R.ts && p == 0 && tid == 0) *RLT(bi, 0) = gtimer();
#endif
        // every lane warp has taken its records of batch bi - NREC (their buffer is reused)
        if (bi >= ROLES_NREC) {
            if (tid == 0) roles_wait_geq(&consumed[bi % ROLES_NREC], (bi / ROLES_NREC) * LW);
            __syncthreads();
        }
        // the range's SA indices and lengths into shared memory: bulk async
        // copies (TMA engine) of their 16-byte aligned cover, the few elements
        // past its last whole 16 bytes by plain loads; or (arrays not 16-byte
        // aligned) loads by all threads
        const uint32_t hs = r0 & 3u, hl = r0 & 7u;
        uint32_t *sav = raw_sa + hs;                       // sav[i - r0] = SA of packet i
        uint16_t *lenv = raw_len + hl;                     // lenv[i - r0] = its length
        if (Q.stage) {
            const uint32_t nbs = r1 > r0 ? ((r1 - r0 + hs) * 4u) & ~15u : 0u;
            const uint32_t nbl = r1 > r0 ? ((r1 - r0 + hl) * 2u) & ~15u : 0u;
            if (tid == 0) {
                const uint32_t mb = smem_u32(mbar);
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(nbs + nbl)
                             : "memory");
                const uint8_t *gs = reinterpret_cast<const uint8_t *>(B.sa_idx + (r0 - hs));
                const uint8_t *gl = reinterpret_cast<const uint8_t *>(B.in_len + (r0 - hl));
                for (uint32_t o = 0; o < nbs; o += 16384u)
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(smem_u32(raw_sa) + o), "l"(gs + o), "r"(min(16384u, nbs - o)), "r"(mb)
                                 : "memory");
                for (uint32_t o = 0; o < nbl; o += 16384u)
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(smem_u32(raw_len) + o), "l"(gl + o), "r"(min(16384u, nbl - o)), "r"(mb)
                                 : "memory");
            }
            // the tails (< 4 SA indices, < 8 lengths)
            for (uint32_t i = r0 - hs + nbs / 4u + tid; i < r1; i += F_THREADS) raw_sa[i - (r0 - hs)] = B.sa_idx[i];
            for (uint32_t i = r0 - hl + nbl / 2u + tid; i < r1; i += F_THREADS)
                raw_len[i - (r0 - hl)] = B.in_len[i];
            __syncthreads();
            tables_bulk_wait(mbar, (bi - (Q.boot ? 1u : 0u)) & 1u);   // (one phase per staged batch)
        } else {
            for (uint32_t i = r0 + tid; i < r1; i += F_THREADS) {
                sav[i - r0] = B.sa_idx[i];
                lenv[i - r0] = B.in_len[i];
            }
            __syncthreads();
        }
        // A. validity, the packet's rank among the warp's earlier packets of its
        //    SA (rounds of 32 in index order, match groups within a round)
        for (uint32_t g0 = w0; g0 < w1; g0 += 32u * NBA_ROLES_AG) {
            uint32_t s[NBA_ROLES_AG], D[NBA_ROLES_AG];
#pragma unroll
            for (uint32_t k = 0; k < NBA_ROLES_AG; k++) {
                const uint32_t i = g0 + 32u * k + lane;
                const bool in = i < w1;
                s[k] = in ? sav[i - r0] : INVALID_SA;
                D[k] = in ? (uint32_t)lenv[i - r0] : 0u;
            }
#pragma unroll
            for (uint32_t k = 0; k < NBA_ROLES_AG; k++) {
                if (g0 + 32u * k >= w1) break;                       // (warp-uniform)
                const uint32_t i = g0 + 32u * k + lane;
                const bool in = i < w1;
                const bool cand = in && s[k] < n_sa && D[k] >= MIN_D && D[k] <= MAX_D;
                // lanes with the same SA (valid ones; SA < 2048): match by ballots
                // over the 11 SA bits and the validity bit
                const uint32_t key = cand ? s[k] : 0x800u;
                uint32_t peers = 0xffffffffu;
                if (NBA_ROLES_MATCH) {
                    peers = __match_any_sync(0xffffffffu, key);
                } else {
#pragma unroll
                    for (uint32_t bit = 0; bit < 12u; bit++) {
                        const bool on = (key >> bit) & 1u;
                        const uint32_t m = __ballot_sync(0xffffffffu, on);
                        peers &= on ? m : ~m;
                    }
                }
                const uint32_t leader = (uint32_t)__ffs(peers) - 1u;
                uint32_t c0 = (cand && lane == leader) ? (uint32_t)mycnt[s[k]] : 0u;
                c0 = __shfl_sync(0xffffffffu, c0, leader);
                if (cand) {
                    rank[i - r0] = (uint16_t)(c0 + __popc(peers & lanemask_lt()));
                    if (lane == leader) mycnt[s[k]] = (uint16_t)(c0 + __popc(peers));
                }
                if (in && !cand) sav[i - r0] = 0xffffffffu;    // dropped: no number
            }
        }
        __syncthreads();
        if (Q.sorted)
            roles_sort_slots(reinterpret_cast<uint4 *>(Q.rec) + (size_t)(bi % ROLES_NREC) * Lc * 512u, Q.cum,
                             lenv, sav, sorth, r0, n, ppc, cbeg, cend);
#if NBA_ROLES_TRACE
        if (R.ts && p == 0 && tid == 0) *RLT(bi, 1) = gtimer();
#endif
        // B. exclusive prefix of the warps' counts per SA; this sequencer's totals
        uint32_t *ptot = Q.ptot + (size_t)(bi & 1u) * P * n_sa;
        for (uint32_t s = tid; s < n_sa; s += F_THREADS) {
            uint32_t run = 0;
#pragma unroll
            for (uint32_t w = 0; w < 16u; w++) {
                const uint32_t c = cnt[w * ROLES_MAX_SA + s];
                cnt[w * ROLES_MAX_SA + s] = (uint16_t)run;
                run += c;
            }
            ptot[(size_t)p * n_sa + s] = run;
        }
        __syncthreads();
#if NBA_ROLES_TRACE
        if (R.ts && p == 0 && tid == 0) *RLT(bi, 2) = gtimer();
#endif
        if (tid == 0) {
            __threadfence();
            roles_red_rel(pbar, 1u);
            roles_wait_geq(pbar, (bi + 1u) * P);
        }
        __syncthreads();
#if NBA_ROLES_TRACE
        if (R.ts && p == 0 && tid == 0) *RLT(bi, 3) = gtimer();
#endif
        // C. per SA: its sequence number before this sequencer's range, and
        //    after the batch (saturating: a packet that would pass 2^32 - 1 is
        //    dropped and consumes nothing)
        for (uint32_t s = tid; s < n_sa; s += F_THREADS) {
            uint32_t before = 0, all = 0;
            for (uint32_t q = 0; q < P; q++) {
                const uint32_t v = __ldcg(&ptot[(size_t)q * n_sa + s]);
                before += q < p ? v : 0u;
                all += v;
            }
            const unsigned long long sq = seqs[s];
            start[s] = sq + before;
            seqs[s] = (uint32_t)min(sq + all, 0xffffffffull);
        }
        __syncthreads();
#if NBA_ROLES_TRACE
        if (R.ts && p == 0 && tid == 0) *RLT(bi, 4) = gtimer();
#endif
        // D. the records (the sequence number, 0 = drop): by packet index, or
        //    (sorted mode) {q, packet} at the packet's lane slot
        uint32_t *rec = Q.rec + (size_t)(bi % ROLES_NREC) * Lc * 512u * (Q.sorted ? 4u : 1u);   // (uint4 records)
#pragma unroll 4
        for (uint32_t g0 = w0; g0 < w1; g0 += 32u) {
            const uint32_t i = g0 + lane;
            if (i < w1) {
                const uint32_t s = sav[i - r0];
                uint32_t r = 0u;
                if (s != 0xffffffffu) {
                    const unsigned long long q =
                        start[s] + mycnt[s] + (unsigned long long)rank[i - r0] + 1ull;
                    r = q <= 0xffffffffull ? (uint32_t)q : 0u;
                }
                if (Q.sorted) {
                    // {q, packet | D << 9 | SA << 20 (D, SA: valid packets only), in_off, out_off}:
                    // the lane needs no load of the packet's fields
                    const uint32_t c = i / ppc;
                    const uint32_t io = B.in_off[i], oo = B.out_off[i];
                    const uint32_t y = (i - c * ppc) | (s != 0xffffffffu ? ((uint32_t)B.in_len[i] << 9) | (s << 20) : 0u);
                    reinterpret_cast<uint4 *>(rec)[(size_t)c * 512u + lenv[i - r0]] = make_uint4(r, y, io, oo);
                    if (s != 0xffffffffu) prefetch_l2(B.in_buf + io);   // its payload's first line
                } else {
                    rec[i] = r;
                }
            }
        }
        __syncwarp();
        for (uint32_t s = lane; s < n_sa; s += 32u) mycnt[s] = 0;   // (the warp's own row)
        __syncthreads();
        if (tid == 0) {
            __threadfence();
            roles_red_rel(&ready[bi % ROLES_NREC], 1u);
#if NBA_ROLES_TRACE
            if (R.ts && p == 0) *RLT(bi, 5) = gtimer();
#endif
        }
    }
    if (p == 0)
        for (uint32_t s = tid; s < n_sa; s += F_THREADS) T.seq[s] = seqs[s];
}

// A lane CTA's counters into the device counters (as fused_body).
__device__ __forceinline__ void roles_lane_counters(const DevWork &W, FusedLo &L, unsigned long long c_ok,
                                                    unsigned long long c_drop, unsigned long long c_in,
                                                    unsigned long long c_out)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31u;
    if (tid < 4) L.cnt[tid] = 0ull;
    __syncthreads();
    const unsigned long long s0 = warp_sum_u64(c_ok), s1 = warp_sum_u64(c_drop);
    const unsigned long long s2 = warp_sum_u64(c_in), s3 = warp_sum_u64(c_out);
    if (lane == 0) {
        if (s0) atomicAdd(&L.cnt[0], s0);
        if (s1) atomicAdd(&L.cnt[1], s1);
        if (s2) atomicAdd(&L.cnt[2], s2);
        if (s3) atomicAdd(&L.cnt[3], s3);
    }
    __syncthreads();
    if (tid < 4 && L.cnt[tid]) atomicAdd(&W.counters[tid], L.cnt[tid]);
}

__device__ __forceinline__ void roles_lanes(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                                            const RingRun &R, const RolesBufs &Q, uint8_t *smem, uint32_t c)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    const uint32_t P = Q.npro, Lc = gridDim.x - P, n_sa = T.n_sa;
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
    // the ring's slot table in shared memory (the per-packet arrays L.sa ..
    // L.aux1 are free in this form): a slot's arguments are read at every
    // batch, and from global memory that load sat on the lanes' critical path
    constexpr uint32_t SLOT_CACHE = (uint32_t)((7u * F_SUPER * sizeof(uint32_t)) / sizeof(BatchArgs));
    static_assert(sizeof(BatchArgs) % 4 == 0, "slot copy by words");
    BatchArgs *sc = reinterpret_cast<BatchArgs *>(&L.sa[0]);
    const bool cached = R.n_slots <= SLOT_CACHE;
    tables_stage(tabs, T, &L.tbar, true);
    const uint32_t *ready = Q.ctl;
    uint32_t *consumed = Q.ctl + ROLES_NREC;
    const uint32_t jpos = lane * 16u + warp;         // position in the CTA's packet range
    unsigned long long c_ok = 0, c_drop = 0, c_in = 0, c_out = 0;
    // The lane's packet fields (batch inputs: SA, length, offsets) are known
    // before its record (the sequence number): loaded one batch ahead, so that
    // the SA line load and the round-key expansion run before the record is
    // needed.  Its payload's first line goes into L2 one batch ahead too.
    struct Fields { uint32_t i, sa, D, inoff, outoff; bool have; };
    const BatchArgs *sl = slots;                     // -> the shared-memory copy below
    auto fields_of = [&](uint32_t bi) {
        Fields f = {0u, INVALID_SA, 0u, 0u, 0u, false};
        if (bi >= R.n_batches) return f;
        const BatchArgs &B = sl[(R.first + bi) % R.n_slots];
        const uint32_t n = B.n, ppc = (n + Lc - 1u) / Lc;
        f.i = c * ppc + jpos;
        f.have = jpos < ppc && f.i < n;
        if (f.have) {
            f.sa = B.sa_idx[f.i];
            f.D = B.in_len[f.i];
            f.inoff = B.in_off[f.i];
            f.outoff = B.out_off[f.i];
        }
        return f;
    };
    auto candidate = [&](const Fields &g) {   // the oracle's step 1 (A15)
        return g.have && g.sa < n_sa && g.D >= MIN_D && g.D <= MAX_D;
    };
    // batch 0's fields from the slot array itself (loads in flight across the
    // bootstrap, in which every CTA numbers batch 0 while the T-table copy
    // lands); the bootstrap also returns the packet SA's counter, read between
    // its barriers (sequencer 0 may finish a short run and write it back after
    // them); then the slot table into shared memory
    Fields f = fields_of(0u);
    const Fields f0 = f;
    const uint32_t seq0 = Q.boot ? roles_boot0(T, slots, R, Q, candidate(f) ? f.sa : INVALID_SA) : 0u;
    if (cached)
        for (uint32_t k = tid; k < R.n_slots * (uint32_t)(sizeof(BatchArgs) / 4); k += F_THREADS)
            reinterpret_cast<uint32_t *>(sc)[k] = reinterpret_cast<const uint32_t *>(slots)[k];
    __syncthreads();
    if (cached) sl = sc;
    tables_bulk_wait(&L.tbar, 0u);
    // experiment (NBA_ROLES_WARM 1 / 2 / 3: all warps / warp 0 / warps 0-3 of
    // each lane CTA): iteration -1 runs the batch-0 code path on a dummy packet
    // (SA 0, the lane's length up to 114 bytes, read from the T-table image,
    // written to a per-CTA scratch line) through the same call sites, during
    // the sequencers' batch 0 -- the first pass over the lane code in a launch
    // is ~1.5x slower than the next ones
    const bool warm_me = cached && R.n_slots < SLOT_CACHE &&
                         (NBA_ROLES_WARM == 1 || NBA_ROLES_WARM == 4 || (NBA_ROLES_WARM == 2 && warp == 0) ||
                          (NBA_ROLES_WARM == 3 && warp < 4u));
    if (NBA_ROLES_WARM && cached && R.n_slots < SLOT_CACHE && tid == 0) {
        BatchArgs bw = sl[R.first % R.n_slots];
        bw.in_buf = reinterpret_cast<const uint8_t *>(T.timg);
        bw.out_buf = Q.scratch + (size_t)c * 256u;
        sc[R.n_slots] = bw;
    }
    if (NBA_ROLES_WARM) __syncthreads();
    if (warm_me) f = Fields{0u, 0u, NBA_ROLES_WARM_D ? NBA_ROLES_WARM_D : (f.have ? min(max(f.D, MIN_D), 114u) : 50u),
                            0u, 14u, true};
    else if (f.have) prefetch_l2(sl[R.first % R.n_slots].in_buf + f.inoff);
    // batch bi's record when it was read ahead (at the end of iteration bi - 1,
    // from a poll issued during it): neither the poll nor the record load then
    // waits on the critical path
    uint32_t q = 0u, rv_next = 0u;
    bool got = false;
    PktPre pp_ahead = {};                  // NBA_ROLES_SAL_AHEAD: the next packet's SA line
    bool have_ahead = false;
    for (int32_t bs = warm_me ? -1 : 0; bs < (int32_t)R.n_batches; bs++) {
        const bool dummy = bs < 0;
        const uint32_t bi = dummy ? 0u : (uint32_t)bs;
        const BatchArgs &B = dummy ? sc[R.n_slots] : sl[(R.first + bi) % R.n_slots];
        const Fields fn = dummy ? f0 : fields_of(bi + 1u);
        const bool cand = candidate(f);
        PktPre pp = {};
        if (NBA_ROLES_SAL_AHEAD && cand && have_ahead) {
            pp = pp_ahead;                                 // loaded at the end of the last iteration
            expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
        } else if (cand) {
            if (NBA_ROLES_RK_ASYNC) {
                // round keys 3..10 copied from the SA's schedule (cp.async into the
                // lane's own slots), 1..2 from its SA line: no expansion chain
                rk_async_issue(T.rk, f.sa, L, H, tid);
                pp = load_pkt_pre(T, B.in_buf, f.sa, f.inoff, true, 0u);
                ldg_nc_v8(&T.sal[(size_t)f.sa * SAL_U4 + 6], pp.r1, pp.r2);
            } else {
                pp = load_pkt_pre(T, B.in_buf, f.sa, f.inoff, true, 0u);
                expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
            }
        }
        if (dummy) {
            q = 1u;
        } else if (Q.boot && bi == 0u) {
            q = cand ? roles_boot_q(Q, B, f.i, f.sa, seq0) : 0u;    // (no record for batch 0)
        } else if (!got) {
#if NBA_ROLES_TRACE
            if (R.ts && c == 0 && tid == 0) *RLT(bi, 6) = gtimer();
#endif
            roles_lane_wait(&ready[bi % ROLES_NREC], (bi / ROLES_NREC + 1u) * P);
#if NBA_ROLES_TRACE
            if (R.ts && c == 0 && tid == 0) *RLT(bi, 7) = gtimer();
#endif
            q = cand ? __ldcg(&Q.rec[(size_t)(bi % ROLES_NREC) * Lc * 512u + f.i]) : 0u;
        }
        if (!dummy) roles_lane_consumed(&consumed[bi % ROLES_NREC], q);
        if (!dummy && lane == 0 && bi + 1u < R.n_batches)
            rv_next = roles_ld_relaxed(&ready[(bi + 1u) % ROLES_NREC]);
        if (NBA_ROLES_RK_ASYNC && cand) rk_async_wait();
        if (f.have) {
            if (q != 0u) {
                // (warm-up mode 4: warp groups enter the code at the CTR precompute,
                // the AES step, the SHA-1 block, the tail)
                const uint32_t g = warp & 3u;
                const uint32_t skip = (NBA_ROLES_WARM == 4 && dummy) ? (g == 0u ? 0u : g == 1u ? 1u : g == 2u ? 3u : 11u)
                                                                     : 0u;
#if NBA_ROLES_TRACE
                // lane timelines of batches 0..3 in lane CTAs 0..3: esp_packet start / end
                unsigned long long *lt = (R.ts && c < 4u && bi < 4u && !dummy)
                    ? R.ts + 1u + 9u * R.n_batches + ((size_t)(bi * 4u + c) * 512u + tid) * 2u : nullptr;
                if (lt) lt[0] = gtimer();
#endif
                esp_packet(T, B, L, H, lane4r, tid, f.sa, f.D | INFO_OK, q, f.inoff, f.outoff, pp, nullptr,
                           nullptr, 0u, skip);
#if NBA_ROLES_TRACE
                if (lt) lt[1] = gtimer();
#endif
                if (dummy) {
                    f = fn;
                    if (f.have) prefetch_l2(sl[R.first % R.n_slots].in_buf + f.inoff);
                    continue;
                }
                // (NBA_ROLES_SAL_L1) the next packet's SA line into L1 right away
                if (NBA_ROLES_SAL_L1 && candidate(fn)) {
                    const uint4 *ln = T.sal + (size_t)fn.sa * SAL_U4;
                    asm volatile("prefetch.global.L1 [%0];" ::"l"(ln));
                    asm volatile("prefetch.global.L1 [%0];" ::"l"(ln + 2));
                }
                const uint32_t Lp = 48u + esp_C(f.D);
                B.out_len[f.i] = (uint16_t)Lp;
                c_ok++;
                c_in += f.D;
                c_out += Lp;
            } else {
                B.out_len[f.i] = 0;
                c_drop++;
            }
        }
        // the next packet's payload line into L2 (its offset has arrived by now)
        if (fn.have) prefetch_l2(sl[(R.first + bi + 1u) % R.n_slots].in_buf + fn.inoff);
        // (NBA_ROLES_SAL_AHEAD) the next packet's SA line, in flight across the loop's tail
        have_ahead = false;
        if (NBA_ROLES_SAL_AHEAD && candidate(fn)) {
            pp_ahead = load_pkt_pre(T, sl[(R.first + bi + 1u) % R.n_slots].in_buf, fn.sa, fn.inoff, true, 0u);
            have_ahead = true;
        }
        if (R.ts && lane == 0) atomicMax(&R.ts[1u + bi], gtimer());
        // the next batch's record, if its sequencers had published it when
        // lane 0's poll (issued above) read the count
        got = false;
        if (bi + 1u < R.n_batches) {
            const uint32_t rv = __shfl_sync(0xffffffffu, rv_next, 0);
            if ((int32_t)(rv - ((bi + 1u) / ROLES_NREC + 1u) * P) >= 0) {
                q = candidate(fn) ? __ldcg(&Q.rec[(size_t)((bi + 1u) % ROLES_NREC) * Lc * 512u + fn.i]) : 0u;
                got = true;
            }
        }
        f = fn;
    }
    roles_lane_counters(W, L, c_ok, c_drop, c_in, c_out);
}

// Lane CTA, sorted mode (mixed-length rings): the record at the thread's own
// lane slot names its packet {q, packet in the CTA's range} -- the packet's
// fields come in the record: {q, j | D << 9 | SA << 20, in_off, out_off} --
// and a fence precedes the "consumed"
// count: a packet slot may go to a different lane in a later batch of the
// same ring slot, so this warp's earlier output stores must be visible before
// the sequencers can publish a batch that reuses them (ring_create takes this
// mode only with n_slots > ROLES_NREC: that batch is at least NREC + 1 later).
__device__ __forceinline__ void roles_lanes_sorted(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                                                   const RingRun &R, const RolesBufs &Q, uint8_t *smem,
                                                   uint32_t c)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31u;
    const uint32_t P = Q.npro, Lc = gridDim.x - P, n_sa = T.n_sa;
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
    constexpr uint32_t SLOT_CACHE = (uint32_t)((7u * F_SUPER * sizeof(uint32_t)) / sizeof(BatchArgs));
    BatchArgs *sc = reinterpret_cast<BatchArgs *>(&L.sa[0]);
    const bool cached = R.n_slots <= SLOT_CACHE;
    if (cached)
        for (uint32_t k = tid; k < R.n_slots * (uint32_t)(sizeof(BatchArgs) / 4); k += F_THREADS)
            reinterpret_cast<uint32_t *>(sc)[k] = reinterpret_cast<const uint32_t *>(slots)[k];
    const BatchArgs *sl = cached ? sc : slots;
    tables_stage(tabs, T, &L.tbar, true);
    __syncthreads();
    tables_bulk_wait(&L.tbar, 0u);
    const uint32_t *ready = Q.ctl;
    uint32_t *consumed = Q.ctl + ROLES_NREC;
    const uint4 *rec = reinterpret_cast<const uint4 *>(Q.rec);
    unsigned long long c_ok = 0, c_drop = 0, c_in = 0, c_out = 0;
    uint4 r = make_uint4(0u, 0xffffffffu, 0u, 0u);
    uint32_t rv_next = 0u;
    bool got = false;
    for (uint32_t bi = 0; bi < R.n_batches; bi++) {
        const BatchArgs &B = sl[(R.first + bi) % R.n_slots];
        if (!got) {
            roles_lane_wait(&ready[bi % ROLES_NREC], (bi / ROLES_NREC + 1u) * P);
            r = __ldcg(&rec[((size_t)(bi % ROLES_NREC) * Lc + c) * 512u + tid]);
        }
        const bool have = r.y != 0xffffffffu;
        const uint32_t i = c * ((B.n + Lc - 1u) / Lc) + (have ? (r.y & 0x1ffu) : 0u);
        // the packet's fields come with its record (q != 0: a valid packet)
        const bool cand = have && r.x != 0u;
        const uint32_t sa = r.y >> 20, D = (r.y >> 9) & 0x7ffu, inoff = r.z, outoff = r.w;
        PktPre pp = {};
        if (cand) {
            pp = load_pkt_pre(T, B.in_buf, sa, inoff, true, 0u);
            expand_key_lane(lane4r, pp.r0, pp.r1, pp.r2, L, H, tid);
        }
        __threadfence();                                // this warp's earlier outputs (see above)
        roles_lane_consumed(&consumed[bi % ROLES_NREC], r.x);
        if (lane == 0 && bi + 1u < R.n_batches) rv_next = roles_ld_relaxed(&ready[(bi + 1u) % ROLES_NREC]);
        if (have) {
            if (r.x != 0u) {
                esp_packet<true>(T, B, L, H, lane4r, tid, sa, D | INFO_OK, r.x, inoff, outoff, pp, nullptr);
                const uint32_t Lp = 48u + esp_C(D);
                B.out_len[i] = (uint16_t)Lp;
                c_ok++;
                c_in += D;
                c_out += Lp;
            } else {
                B.out_len[i] = 0;
                c_drop++;
            }
        }
        if (R.ts && lane == 0) atomicMax(&R.ts[1u + bi], gtimer());
        got = false;
        if (bi + 1u < R.n_batches) {
            const uint32_t rv = __shfl_sync(0xffffffffu, rv_next, 0);
            if ((int32_t)(rv - ((bi + 1u) / ROLES_NREC + 1u) * P) >= 0) {
                r = __ldcg(&rec[((size_t)((bi + 1u) % ROLES_NREC) * Lc + c) * 512u + tid]);
                got = true;
            }
        }
    }
    roles_lane_counters(W, L, c_ok, c_drop, c_in, c_out);
}

__global__ void __launch_bounds__(F_THREADS, 1)
k_fused_ring_roles(DevTable T, DevWork W, const BatchArgs *slots, RingRun R, RolesBufs Q)
{
    extern __shared__ __align__(16) uint8_t smem[];
    if (R.n_batches == 0) return;
    if (R.ts && blockIdx.x == 0 && threadIdx.x == 0) R.ts[0] = gtimer();
    if (blockIdx.x < Q.npro) roles_sequencer(T, slots, R, Q, smem, blockIdx.x);
    else if (Q.sorted) roles_lanes_sorted(T, W, slots, R, Q, smem, blockIdx.x - Q.npro);
    else roles_lanes(T, W, slots, R, Q, smem, blockIdx.x - Q.npro);
    // leave; the last CTA out zeroes the hand-off counters for the next launch
    __syncthreads();
    if (threadIdx.x == 0) {
        if (blockIdx.x == 0) atomicAdd(&W.counters[4], (unsigned long long)R.n_batches);
        __threadfence();
        const uint32_t t = atomicAdd(&Q.ctl[2u * ROLES_NREC + 1u], 1u);
        if (t == gridDim.x - 1u) {
            __threadfence();
            for (uint32_t k = 0; k < ROLES_CTL_WORDS; k++) atomicExch(&Q.ctl[k], 0u);
        }
    }
}

bool fused_roles_ok(uint32_t n, uint32_t n_sa, int grid, uint32_t npro)
{
    if (npro == 0 || grid <= (int)npro || n == 0 || n_sa == 0 || n_sa > ROLES_MAX_SA) return false;
    const uint32_t Lc = (uint32_t)grid - npro, ppc = (n + Lc - 1u) / Lc;
    // a sequencer's range: its ceil(Lc / npro) lane CTAs' packets
    return ppc <= 512u && ((Lc + npro - 1u) / npro) * ppc <= ROLES_RPP_MAX;
}

cudaError_t launch_fused_ring_roles(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                                    const RingRun &R, const RolesBufs &Q, int grid, cudaStream_t st)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(F_THREADS);
    cfg.dynamicSmemBytes = F_SMEM;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;   // the roles wait on each other: co-resident
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_fused_ring_roles, T, W, slots, R, Q);
}

cudaError_t launch_fused_ring_free(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                                   const RingRun &R, uint16_t *hist_b, int grid, cudaStream_t st)
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
    return cudaLaunchKernelEx(&cfg, k_fused_ring_free, T, W, slots, R, hist_b);
}

cudaError_t launch_fused_ring_pipe(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                                   const RingRun &R, uint16_t *hist_b, int grid, cudaStream_t st)
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
    return cudaLaunchKernelEx(&cfg, k_fused_ring_pipe, T, W, slots, R, hist_b);
}

bool fused_pipe_ok(uint32_t n, int grid)
{
    // pipe_scan_rows covers rows of up to 8 x 20 = 160 CTAs
    return n > 0 && grid <= 160 && fused_ppc(n, grid) <= PIPE_MAX_PPC;
}

int fused_grid(int num_sms) { return num_sms; }



bool fused_merged_ok(uint32_t n, int grid)
{
    return fused_ppc(n, grid) <= (uint32_t)F_SUPER;
}

cudaError_t launch_fused(const DevTable &T, const DevWork &W, const BatchArgs &B, int grid,
                         bool merged, uint32_t *bar_base, uint32_t *epoch, cudaStream_t st)
{
    uint32_t ppc = fused_ppc(B.n, grid);
    uint32_t g = (B.n + ppc - 1) / ppc;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(g);
    cfg.blockDim = dim3(F_THREADS);
    cfg.dynamicSmemBytes = F_SMEM;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    static const bool no_coop = std::getenv("NBA_IPSEC_NO_COOP") != nullptr;   // A/B only
    if (merged) {
        // grid barriers inside: the driver must make all CTAs co-resident
        attr[0].id = cudaLaunchAttributeCooperative;
        attr[0].val.cooperative = no_coop ? 0 : 1;
    } else {
        attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[0].val.programmaticStreamSerializationAllowed = 1;
    }
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    // the one-kernel path keeps its barrier base and 31-bit batch epoch on the
    // device (W.ctl), so a launch carries no per-batch host state and can be
    // replayed from a CUDA graph; the host copies only count launches
    (void)bar_base;
    (void)epoch;
    return merged ? cudaLaunchKernelEx(&cfg, k_fused<true>, T, W, B, ppc, 0u, 0u)
                  : cudaLaunchKernelEx(&cfg, k_fused<false>, T, W, B, ppc, 0u, 0u);
}

cudaError_t launch_fused_ring(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                              const RingRun &R, uint16_t *hist_b, int grid, cudaStream_t st)
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
    return cudaLaunchKernelEx(&cfg, k_fused_ring, T, W, slots, R, hist_b);
}

cudaError_t setup_fused_attributes()
{
    cudaError_t e0 = cudaFuncSetAttribute(k_fused_ring, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)F_SMEM);
    if (e0 != cudaSuccess) return e0;
    e0 = cudaFuncSetAttribute(k_fused_ring_pipe, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)F_SMEM);
    if (e0 != cudaSuccess) return e0;
    e0 = cudaFuncSetAttribute(k_fused_ring_free, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)F_SMEM);
    if (e0 != cudaSuccess) return e0;
    e0 = cudaFuncSetAttribute(k_fused_ring_roles, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)F_SMEM);
    if (e0 != cudaSuccess) return e0;
    cudaError_t e = cudaFuncSetAttribute(k_fused<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)F_SMEM);
    if (e != cudaSuccess) return e;
    return cudaFuncSetAttribute(k_fused<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)F_SMEM);
}

}  // namespace nba
