// k_fused.cu -- rows a2..a5 in ONE persistent kernel (the
// datablock-reuse / copy-coalescing optimisation NBA left as future work,
// PAPER.md:329 and :345).
//
// One 768-thread CTA per SM shares one 128 KB bank-replicated T-table image.
// Each CTA owns a contiguous packet range and walks it in super-rounds of up
// to F_SUPER packets:
//   1. all threads, one packet each: validity, sizes, ESP sequence number (from
//      the prologue's per-SA ranks), a CTA-local counting sort by SHA-1 length
//      (longest first), the per-packet CTR-mode precomputation of AES rounds
//      1-2 (all counter blocks of a packet share 15 of 16 input bytes, so round
//      1 needs 1 table lookup and round 2 needs 4 instead of 16 each), and a
//      shared-memory copy of round keys 3..10;
//   2. dynamic roles: every warp claims 32-pair AES chunks (a thread encrypts
//      TWO consecutive 16-byte blocks of one packet: payload read straight from
//      the caller's buffer, pad / trailer appended, RFC 3686 keystream XORed,
//      ciphertext stored directly at its final place in the output slot with
//      destination-aligned 16-byte stores, neighbouring lanes exchanging the
//      unaligned seam with a shuffle), and claims the next HMAC group (32
//      packets, one lane each) as soon as an mbarrier says all of the group's
//      blocks are encrypted: outer IPv4 + ESP header, HMAC-SHA1-96 over
//      SPI..ciphertext from the SA's precomputed midstates (ciphertext read
//      back from L2), ICV appended.
// AES (shared-memory LSU bound) and SHA-1 (ALU bound) run concurrently on every
// SM; every payload byte is read from HBM once and written once.
//
// Shared-memory layout: the T-tables sit at a 64 KB-aligned shared-window
// address, so a single PRMT forms the complete LDS address of a lookup
// (byte r of the state word in bits 8..15, lane*4 in bits 0..7, the table base
// in bits 16..31) -- no address add per lookup.  The rest of the state lives
// below (FusedLo) and above (FusedHi) the tables.
#include "aes_round.cuh"
#include "sha1.cuh"

namespace nba {

constexpr int F_WARPS = 24;
constexpr int F_THREADS = 32 * F_WARPS;   // 768 -> up to 80 registers
constexpr int F_SUPER = 512;              // packets per super-round
constexpr int F_GROUPS = F_SUPER / 32;
constexpr int F_MAX_PAIRS = 47;           // ceil(94 blocks / 2)
constexpr int F_CHUNKS = F_SUPER * F_MAX_PAIRS / 32 + 2;

struct FusedLo {
    uint32_t ppref[F_SUPER + 1];   // AES pair prefix in sorted (position) order
    uint16_t perm[F_SUPER];        // position -> packet index in the super-round
    uint16_t sa[F_SUPER];          // by packet index (n_sa <= 65536)
    uint32_t seq[F_SUPER];
    uint32_t info[F_SUPER];        // D | tos << 16 | INFO_OK  (0: dropped)
    uint32_t inoff[F_SUPER];
    uint32_t outoff[F_SUPER];
    uint4 pre0[F_SUPER];           // X0, Z0, Z1, Z2 (CTR precompute)
    uint32_t pre1[F_SUPER];        // Z3
    uint8_t pre2[F_SUPER];         // byte 3 of round-key word rk0.w
    uint4 rkA[4][F_SUPER];         // round keys 3..6, round-major (conflict-free LDS.128)
    uint32_t gneed[F_GROUPS];      // AES pairs per HMAC group
    unsigned long long gbar[F_GROUPS];   // mbarrier per HMAC group
    uint32_t aes_next;             // next 32-pair AES chunk to claim
    uint32_t hmac_next;            // next HMAC group to claim (in order)
    uint32_t bins[NBINS];
    uint32_t scr[32];
    unsigned long long cnt[4];
};

struct FusedHi {
    uint4 rkB[4][F_SUPER];         // round keys 7..10, round-major
    uint16_t chunkpos[F_CHUNKS];   // first position of every 32-pair chunk
};

// Dynamic shared memory: [Lo | pad][tables 128 KB][Hi].  With the usual 1 KB of
// reserved shared memory the tables start at shared address 0x10000.
constexpr uint32_t F_TOFF_MAX = 0xFC00u;
constexpr size_t F_SMEM = F_TOFF_MAX + AES_TABLE_BYTES + sizeof(FusedHi);
static_assert(sizeof(FusedLo) <= F_TOFF_MAX, "FusedLo must fit below the tables");
static_assert(F_SMEM <= 232448, "exceeds 227 KB of shared memory per block");

// -------------------------------------------------------------------- helpers
__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return (uint32_t)__cvta_generic_to_shared(p);
}

template <uint32_t OFF>
__device__ __forceinline__ uint32_t lds_abs(uint32_t a)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(a), "n"(OFF));
    return v;
}

// T-table lookup: table `tbl`, row `row` of state word `reg`; lane4r holds
// lane*4 in bits 0..7 and the 64 KB-aligned table base in bits 16..31.
#define TL(reg, row, tbl)                                                                  \
    lds_abs<((tbl) >> 1) * 0x10000u + ((tbl) & 1u) * 0x80u>(                               \
        __byte_perm((reg), lane4r, 0x7604u | ((row) << 4)))

__device__ __forceinline__ uint32_t trailer_byte_f(uint32_t b, uint32_t D, uint32_t p)
{
    if (b < D + p) return b - D + 1u;
    if (b == D + p) return p;
    if (b == D + p + 1u) return 4u;
    return 0u;
}

// 16 bytes of T = P || pad || p || 4 at byte pos, from the aligned chunks lo, hi
// covering P bytes [pos, pos+16) at offset sh.
__device__ __forceinline__ uint4 payload_finish(uint4 lo, uint4 hi, uint32_t sh, uint32_t D,
                                                uint32_t p, uint32_t pos)
{
    uint4 v = make_uint4(0, 0, 0, 0);
    if (pos < D) {
        v = extract16(lo, hi, sh);
        if (pos + 16 <= D) return v;
    }
#pragma unroll
    for (uint32_t j = 0; j < 16; j++) {
        uint32_t b = pos + j;
        if (b >= D) set_byte(v, j, trailer_byte_f(b, D, p));
    }
    return v;
}

__device__ __forceinline__ uint32_t word_of(uint4 v, uint32_t i)
{
    return i == 0 ? v.x : i == 1 ? v.y : i == 2 ? v.z : v.w;
}

__device__ __forceinline__ void stg_v4(void *p, uint4 v)
{
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
                 "r"(v.w)
                 : "memory");
}

// Bytes [lo, hi) of the 16-byte image v to chunk + [lo, hi); chunk 16-B aligned.
__device__ __forceinline__ void store_chunk_range(uint8_t *chunk, uint4 v, uint32_t lo, uint32_t hi)
{
    if (lo == 0 && hi == 16) {
        stg_v4(chunk, v);
        return;
    }
    uint32_t x = lo;
    while (x < hi) {
        uint32_t w = word_of(v, x >> 2);
        if ((x & 3u) == 0 && x + 4 <= hi) {
            asm volatile("st.global.u32 [%0], %1;" ::"l"(chunk + x), "r"(w) : "memory");
            x += 4;
        } else if ((x & 1u) == 0 && x + 2 <= hi) {
            asm volatile("st.global.u16 [%0], %1;" ::"l"(chunk + x),
                         "h"((unsigned short)(w >> ((x & 3u) * 8u)))
                         : "memory");
            x += 2;
        } else {
            asm volatile("st.global.u8 [%0], %1;" ::"l"(chunk + x),
                         "h"((unsigned short)((w >> ((x & 3u) * 8u)) & 0xffu))
                         : "memory");
            x += 1;
        }
    }
}

// NW little-endian words (4*NW bytes) to an address of any alignment, as
// destination-aligned pieces.
template <int NW>
__device__ __forceinline__ void store_words_unaligned(uint8_t *dst, const uint32_t (&w)[NW])
{
    uintptr_t a = reinterpret_cast<uintptr_t>(dst);
    uint32_t sh = (uint32_t)(a & 15u);
    uint8_t *c0 = reinterpret_cast<uint8_t *>(a & ~(uintptr_t)15);
    constexpr int NC = (NW * 4 + 15) / 16 + 1;
#pragma unroll
    for (int c = 0; c < NC; c++) {
        int s = 16 * c - (int)sh;                  // source byte of chunk byte 0
        uint32_t lo = s < 0 ? (uint32_t)(-s) : 0u;
        int hi_i = NW * 4 - s;
        uint32_t hi = hi_i >= 16 ? 16u : (hi_i < 0 ? 0u : (uint32_t)hi_i);
        if (lo >= hi) continue;
        uint32_t o[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            int sb = s + 4 * k;
            int wi = sb >> 2;                      // floor (sb may be negative)
            uint32_t r = (uint32_t)(sb & 3) * 8u;
            uint32_t a0 = 0, a1 = 0;
#pragma unroll
            for (int q = 0; q < NW; q++) {
                if (q == wi) a0 = w[q];
                if (q == wi + 1) a1 = w[q];
            }
            o[k] = r ? __funnelshift_r(a0, a1, r) : a0;
        }
        store_chunk_range(c0 + 16 * c, make_uint4(o[0], o[1], o[2], o[3]), lo, hi);
    }
}

// 64 message bytes at p (any alignment) as big-endian words; aligned chunks
// wholly at or past `end` are not touched (read as zero).
__device__ __forceinline__ void load_block64_unaligned(uint32_t w[16], const uint8_t *p,
                                                       const uint8_t *end)
{
    uintptr_t a = reinterpret_cast<uintptr_t>(p);
    uintptr_t base = a & ~(uintptr_t)15;
    uintptr_t e = reinterpret_cast<uintptr_t>(end);
    uint32_t sh = (uint32_t)(a & 15u);
    uint4 c[5];
#pragma unroll
    for (int i = 0; i < 5; i++) {
        uintptr_t q = base + 16u * i;
        c[i] = q < e ? *reinterpret_cast<const uint4 *>(q) : make_uint4(0, 0, 0, 0);
    }
    uint32_t v[20] = {c[0].x, c[0].y, c[0].z, c[0].w, c[1].x, c[1].y, c[1].z, c[1].w,
                      c[2].x, c[2].y, c[2].z, c[2].w, c[3].x, c[3].y, c[3].z, c[3].w,
                      c[4].x, c[4].y, c[4].z, c[4].w};
    const uint32_t r = (sh & 3u) * 8u;
#define NBA_LD_CASE(Q)                                                                   \
    _Pragma("unroll") for (int j = 0; j < 16; j++) w[j] =                                \
        bswap32(__funnelshift_r(v[(Q) + j], v[(Q) + j + 1], r));
    switch (sh >> 2) {
    case 0: NBA_LD_CASE(0) break;
    case 1: NBA_LD_CASE(1) break;
    case 2: NBA_LD_CASE(2) break;
    default: NBA_LD_CASE(3) break;
    }
#undef NBA_LD_CASE
}

__device__ __forceinline__ void mbar_init(unsigned long long *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
                 : "memory");
}

__device__ __forceinline__ void mbar_inval(unsigned long long *bar)
{
    asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// release: the arriving thread's earlier stores (and, through __syncwarp, its
// warp's) are visible to a thread that observes the phase completion
__device__ __forceinline__ void mbar_arrive(unsigned long long *bar, uint32_t count)
{
    asm volatile("{\n\t.reg .b64 st;\n\t"
                 "mbarrier.arrive.release.cta.shared::cta.b64 st, [%0], %1;\n\t}" ::"r"(smem_u32(bar)),
                 "r"(count)
                 : "memory");
}

// blocking wait (hardware-suspended between polls) for phase 0 to complete
__device__ __forceinline__ void mbar_wait_parity0(unsigned long long *bar)
{
    uint32_t done = 0;
    while (!done) {
        asm volatile("{\n\t.reg .pred p;\n\t"
                     "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], 0, 1000000;\n\t"
                     "selp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(done)
                     : "r"(smem_u32(bar))
                     : "memory");
    }
}

__device__ __forceinline__ bool mbar_test_parity0(unsigned long long *bar)
{
    uint32_t done;
    asm volatile("{\n\t.reg .pred p;\n\t"
                 "mbarrier.test_wait.parity.acquire.cta.shared::cta.b64 p, [%1], 0;\n\t"
                 "selp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(done)
                 : "r"(smem_u32(bar))
                 : "memory");
    return done != 0;
}

// ------------------------------------------------- AES: 32 lanes x 2 blocks
__device__ __forceinline__ void aes_pair_chunk(const BatchArgs &B, FusedLo &L, FusedHi &H,
                                               uint32_t lane4r, uint32_t c, uint32_t total_pairs,
                                               uint32_t lane, unsigned long long *dbg)
{
    long long ck0 = clock64();
    const uint32_t q = c * 32u + lane;
    const bool act = q < total_pairs;
    // inactive lanes repeat the last pair so the rounds stay warp-uniform
    const uint32_t qq = act ? q : total_pairs - 1u;
    uint32_t pos = H.chunkpos[c];
    while (L.ppref[pos + 1] <= qq) pos++;
    const uint32_t kp = qq - L.ppref[pos];
    const uint32_t pk = L.perm[pos];
    const uint32_t D = L.info[pk] & 0x7ffu;
    const uint32_t C = esp_C(D);
    const uint32_t k0 = 2u * kp;

    // raw payload loads: P bytes [16*k0, 16*k0 + 32), consumed after the rounds
    const uint8_t *src = B.in_buf + L.inoff[pk];
    const uintptr_t a = reinterpret_cast<uintptr_t>(src) + 16u * k0;
    const uintptr_t abase = a & ~(uintptr_t)15;
    const uintptr_t aend = reinterpret_cast<uintptr_t>(src) + D;
    const uint32_t sh = (uint32_t)(a & 15u);
    const uint4 z4 = make_uint4(0, 0, 0, 0);
    const uint4 c0 = (abase < aend) ? ldg_nc_v4(reinterpret_cast<const void *>(abase)) : z4;
    const uint4 c1 = (abase + 16 < aend) ? ldg_nc_v4(reinterpret_cast<const void *>(abase + 16)) : z4;
    const uint4 c2 = (abase + 32 < aend) ? ldg_nc_v4(reinterpret_cast<const void *>(abase + 32)) : z4;

    const uint4 pre = L.pre0[pk];
    const uint32_t Z3 = L.pre1[pk];
    const uint32_t r3 = L.pre2[pk];
    long long ck1 = clock64();
    // rounds 1-2 from the per-packet precompute, two counter blocks (k0+1, k0+2)
    const uint32_t ta = TL(((r3 ^ (k0 + 1u)) << 24), 3, 3) ^ pre.x;
    const uint32_t tb = TL(((r3 ^ (k0 + 2u)) << 24), 3, 3) ^ pre.x;
    uint32_t a0 = TL(ta, 0, 0) ^ pre.y, a1 = TL(ta, 3, 3) ^ pre.z, a2 = TL(ta, 2, 2) ^ pre.w,
             a3 = TL(ta, 1, 1) ^ Z3;
    uint32_t b0 = TL(tb, 0, 0) ^ pre.y, b1 = TL(tb, 3, 3) ^ pre.z, b2 = TL(tb, 2, 2) ^ pre.w,
             b3 = TL(tb, 1, 1) ^ Z3;
    // rounds 3..9 as a rolled loop: keeps the hot code within the instruction cache
    // alongside the SHA-1 compression that other warps run concurrently
#pragma unroll 1
    for (int r = 3; r < 10; r++) {
        const uint4 rk = r < 7 ? L.rkA[r - 3][pk] : H.rkB[r - 7][pk];
        const uint32_t u0 = TL(a0, 0, 0) ^ TL(a1, 1, 1) ^ TL(a2, 2, 2) ^ TL(a3, 3, 3) ^ rk.x;
        const uint32_t u1 = TL(a1, 0, 0) ^ TL(a2, 1, 1) ^ TL(a3, 2, 2) ^ TL(a0, 3, 3) ^ rk.y;
        const uint32_t u2 = TL(a2, 0, 0) ^ TL(a3, 1, 1) ^ TL(a0, 2, 2) ^ TL(a1, 3, 3) ^ rk.z;
        const uint32_t u3 = TL(a3, 0, 0) ^ TL(a0, 1, 1) ^ TL(a1, 2, 2) ^ TL(a2, 3, 3) ^ rk.w;
        const uint32_t v0 = TL(b0, 0, 0) ^ TL(b1, 1, 1) ^ TL(b2, 2, 2) ^ TL(b3, 3, 3) ^ rk.x;
        const uint32_t v1 = TL(b1, 0, 0) ^ TL(b2, 1, 1) ^ TL(b3, 2, 2) ^ TL(b0, 3, 3) ^ rk.y;
        const uint32_t v2 = TL(b2, 0, 0) ^ TL(b3, 1, 1) ^ TL(b0, 2, 2) ^ TL(b1, 3, 3) ^ rk.z;
        const uint32_t v3 = TL(b3, 0, 0) ^ TL(b0, 1, 1) ^ TL(b1, 2, 2) ^ TL(b2, 3, 3) ^ rk.w;
        a0 = u0; a1 = u1; a2 = u2; a3 = u3;
        b0 = v0; b1 = v1; b2 = v2; b3 = v3;
    }
    const uint4 rk = H.rkB[3][pk];
    long long ck2 = clock64();
    // final round: S[x] is byte (j+2)&3 of Tj[x]
#define NBA_FINAL(s0, s1, s2, s3)                                                               \
    ((TL(s0, 0, 2) & 0x000000ffu) | (TL(s1, 1, 3) & 0x0000ff00u) | (TL(s2, 2, 0) & 0x00ff0000u) | \
     (TL(s3, 3, 1) & 0xff000000u))
    const uint32_t p = esp_pad(D);
    const uint4 pt0 = payload_finish(c0, c1, sh, D, p, 16u * k0);
    const uint4 pt1 = payload_finish(c1, c2, sh, D, p, 16u * k0 + 16u);
    uint4 ct0, ct1;
    ct0.x = pt0.x ^ rk.x ^ NBA_FINAL(a0, a1, a2, a3);
    ct0.y = pt0.y ^ rk.y ^ NBA_FINAL(a1, a2, a3, a0);
    ct0.z = pt0.z ^ rk.z ^ NBA_FINAL(a2, a3, a0, a1);
    ct0.w = pt0.w ^ rk.w ^ NBA_FINAL(a3, a0, a1, a2);
    ct1.x = pt1.x ^ rk.x ^ NBA_FINAL(b0, b1, b2, b3);
    ct1.y = pt1.y ^ rk.y ^ NBA_FINAL(b1, b2, b3, b0);
    ct1.z = pt1.z ^ rk.z ^ NBA_FINAL(b2, b3, b0, b1);
    ct1.w = pt1.w ^ rk.w ^ NBA_FINAL(b3, b0, b1, b2);
#undef NBA_FINAL

    // ---- destination-aligned stores of the 32-byte run ct0 || ct1 --------------
    __syncwarp();
    long long ck3 = clock64();
    uint4 prv;   // previous lane's ct1 (the tail of the pair before ours)
    prv.x = __shfl_up_sync(0xffffffffu, ct1.x, 1);
    prv.y = __shfl_up_sync(0xffffffffu, ct1.y, 1);
    prv.z = __shfl_up_sync(0xffffffffu, ct1.z, 1);
    prv.w = __shfl_up_sync(0xffffffffu, ct1.w, 1);
    const uint32_t ppos = __shfl_up_sync(0xffffffffu, pos, 1);
    const uint32_t npos = __shfl_down_sync(0xffffffffu, pos, 1);
    const bool nact = __shfl_down_sync(0xffffffffu, act ? 1u : 0u, 1) != 0;
    if (act) {
        const uint32_t V = min(32u, C - 16u * k0);        // ciphertext bytes of this pair
        const bool prev_same = lane > 0 && ppos == pos && kp > 0;
        const bool next_same = lane < 31 && nact && npos == pos;
        uint8_t *bs = B.out_buf + L.outoff[pk] + 36u + 16u * k0;
        const uint32_t m = (uint32_t)(reinterpret_cast<uintptr_t>(bs) & 15u);
        uint8_t *A = bs - m;
        if (m == 0) {
            store_chunk_range(A, ct0, 0, min(16u, V));
            if (V > 16u) store_chunk_range(A + 16, ct1, 0, V - 16u);
        } else {
            const uint32_t mm = 16u - m;
            store_chunk_range(A, extract16(prv, ct0, mm), prev_same ? 0u : m, min(16u, m + V));
            if (V > mm) store_chunk_range(A + 16, extract16(ct0, ct1, mm), 0, min(16u, V - mm));
            if (!next_same && V > 32u - m)
                store_chunk_range(A + 32, extract16(ct1, z4, mm), 0, V - (32u - m));
        }
    }
    // completion: one release-arrive per (warp, HMAC group) after all lanes' stores
    __syncwarp();
    const uint32_t grp = act ? (pos >> 5) : 0xffffffffu;
    const uint32_t peers = __match_any_sync(0xffffffffu, grp);
    if (act && lane == (uint32_t)(__ffs(peers) - 1)) mbar_arrive(&L.gbar[grp], __popc(peers));
    if (dbg && lane == 0) {
        long long ck4 = clock64();
        dbg[0] = ck1 - ck0; dbg[1] = ck2 - ck1; dbg[2] = ck3 - ck2; dbg[3] = ck4 - ck3;
        dbg[4] = ct0.x ^ ct1.y;   // keep values live
    }
}

// ---------------------------------- HMAC-SHA1-96 of one 32-packet group
__device__ __forceinline__ void hmac_group(const DevTable &T, const BatchArgs &B, FusedLo &L,
                                           uint32_t base, uint32_t g, uint32_t cnt_pk, uint32_t lane)
{
    const uint32_t pos = g * 32u + lane;
    const bool have = pos < cnt_pk;
    const uint32_t pk = have ? L.perm[pos] : 0u;
    const uint32_t info = have ? L.info[pk] : 0u;
    const bool ok = (info & INFO_OK) != 0;
    const uint32_t D = info & 0x7ffu;
    const uint32_t C = ok ? esp_C(D) : 0u;
    const uint32_t Ln = ok ? 48u + C : 0u;
    const uint32_t pkt = base + pk;
    if (ok) {
        const uint32_t sa = L.sa[pk];
        const uint4 hd = __ldg(&T.sahdr[sa]);
        const uint32_t qbe = bswap32(L.seq[pk]);
        uint8_t *o = B.out_buf + L.outoff[pk];
        // outer IPv4 header (reading A13) + ESP header + IV, 36 bytes
        uint32_t hdr[9];
        {
            const uint32_t tos = (info >> 16) & 0xffu;
            const uint32_t src = bswap32(hd.z), dst = bswap32(hd.w);
            uint32_t sum = (0x4500u | tos) + Ln + 0x4000u + ((64u << 8) | 50u) + (src >> 16) +
                           (src & 0xffffu) + (dst >> 16) + (dst & 0xffffu);
            sum = (sum & 0xffffu) + (sum >> 16);
            sum = (sum & 0xffffu) + (sum >> 16);
            const uint32_t cs = ~sum & 0xffffu;
            hdr[0] = 0x45u | (tos << 8) | ((Ln >> 8) << 16) | ((Ln & 0xffu) << 24);
            hdr[1] = 0x00400000u;
            hdr[2] = 64u | (50u << 8) | ((cs >> 8) << 16) | ((cs & 0xffu) << 24);
            hdr[3] = hd.z;
            hdr[4] = hd.w;
            hdr[5] = hd.x;
            hdr[6] = qbe;
            hdr[7] = 0u;
            hdr[8] = qbe;
        }
        store_words_unaligned<9>(o, hdr);
        const uint4 h0 = __ldg(&T.hmid[(size_t)sa * 3 + 0]);
        const uint4 h1 = __ldg(&T.hmid[(size_t)sa * 3 + 1]);
        const uint4 h2 = __ldg(&T.hmid[(size_t)sa * 3 + 2]);
        const uint32_t hin[5] = {h0.x, h0.y, h0.z, h0.w, h1.x};
        const uint32_t hout[5] = {h1.y, h1.z, h1.w, h2.x, h2.y};
        const uint8_t *m0 = o + 20;                 // ESP header: start of the MAC input
        const uint8_t *mend = m0 + 16u + C;
        uint32_t icv[3];
        hmac_sha1_96(hin, hout, C,
                     [&](uint32_t w[16], uint32_t bb) { load_block64_unaligned(w, m0 + 64u * bb, mend); },
                     icv);
        const uint32_t iw[3] = {bswap32(icv[0]), bswap32(icv[1]), bswap32(icv[2])};
        store_words_unaligned<3>(o + 36u + C, iw);
    }
    if (have) B.out_len[pkt] = (uint16_t)Ln;
    __syncwarp();
    const uint32_t s0 = __reduce_add_sync(0xffffffffu, ok ? 1u : 0u);
    const uint32_t s1 = __reduce_add_sync(0xffffffffu, (have && !ok) ? 1u : 0u);
    const uint32_t s2 = __reduce_add_sync(0xffffffffu, ok ? D : 0u);
    const uint32_t s3 = __reduce_add_sync(0xffffffffu, Ln);
    if (lane == 0) {
        atomicAdd(&L.cnt[0], (unsigned long long)s0);
        atomicAdd(&L.cnt[1], (unsigned long long)s1);
        atomicAdd(&L.cnt[2], (unsigned long long)s2);
        atomicAdd(&L.cnt[3], (unsigned long long)s3);
    }
}

// ---------------------------------------------------------------- the kernel
__global__ void __launch_bounds__(F_THREADS, 1)
k_fused(DevTable T, DevWork W, BatchArgs B, uint32_t ppc)
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

    aes_tables_to_smem(tabs, T.te0);
    if (tid < 4) L.cnt[tid] = 0ull;

    const uint32_t p_begin = blockIdx.x * ppc;
    const uint32_t p_end = min(B.n, p_begin + ppc);
    static_assert(F_SUPER <= F_THREADS, "one packet per thread in the metadata phase");

    for (uint32_t base = p_begin; base < p_end; base += F_SUPER) {
        const uint32_t cnt_pk = min((uint32_t)F_SUPER, p_end - base);
        // ---- 1. metadata (thread j <-> packet base + j) ---------------------
        if (tid < NBINS) L.bins[tid] = 0;
        const uint32_t j = tid;
        const uint32_t i = base + j;
        // 1a. everything that does not depend on the prologue (overlaps it
        //     under programmatic dependent launch on the first round)
        uint32_t sa = INVALID_SA, D = 0, inoff = 0, tos = 0, nonce = 0;
        bool cand = false;
        uint4 r0 = make_uint4(0, 0, 0, 0), r1 = r0, r2 = r0;
        if (j < cnt_pk) {
            sa = B.sa_idx[i];
            D = B.in_len[i];
            inoff = B.in_off[i];
            L.outoff[j] = B.out_off[i];
            cand = sa < n_sa && D >= MIN_D && D <= MAX_D;
            if (cand) {
                tos = B.in_buf[inoff + 1];
                const uint4 *rks = T.rk + (size_t)sa * 11u;
                r0 = __ldg(&rks[0]);
                r1 = __ldg(&rks[1]);
                r2 = __ldg(&rks[2]);
                nonce = __ldg(&T.sahdr[sa].y);
#pragma unroll
                for (int r = 0; r < 4; r++) {
                    L.rkA[r][j] = __ldg(&rks[3 + r]);
                    H.rkB[r][j] = __ldg(&rks[7 + r]);
                }
            }
        }
        // Programmatic dependent launch: the prologue's outputs (ranks, per-SA
        // prefixes, seq_prev) are complete and visible after this.
        if (base == p_begin) asm volatile("griddepcontrol.wait;" ::: "memory");
        __syncthreads();   // also publishes the T-tables on the first round
        // 1b. sequence number, drop decision, CTR precompute
        if (j < cnt_pk) {
            uint32_t info = 0, bin = NBINS - 1, q32 = 0;
            if (cand) {
                const unsigned long long q = (unsigned long long)T.seq_prev[sa] + 1ull +
                                             W.hpfx[(size_t)(i / PTILE) * n_sa + sa] + W.lrank[i];
                if (q <= 0xffffffffull) {   // RFC 4303 §3.3.3: never cycle
                    q32 = (uint32_t)q;
                    info = D | (tos << 16) | INFO_OK;
                    bin = hmac_bin(true, esp_C(D));
                    // CTR precompute (FIPS-197 Cipher() rounds 1-2 on the counter block
                    // nonce || 0 || BE32(q) || BE32(k+1), k+1 < 256): only byte 3 of
                    // column 3 varies, so after round 1 only column 0 varies, through
                    // one T3 lookup: t0 = T3[r3 ^ (k+1)] ^ X0, and round 2 is
                    // u_c = T[row(t0)] ^ Z_c with one lookup per column.
                    const uint32_t s0 = nonce ^ r0.x;
                    const uint32_t s1 = r0.y;
                    const uint32_t s2 = bswap32(q32) ^ r0.z;
                    const uint32_t s3 = r0.w;     // byte 3 is XORed with (k+1) per block
                    const uint32_t X0 = TL(s0, 0, 0) ^ TL(s1, 1, 1) ^ TL(s2, 2, 2) ^ r1.x;
                    const uint32_t Y1 = TL(s1, 0, 0) ^ TL(s2, 1, 1) ^ TL(s3, 2, 2) ^ TL(s0, 3, 3) ^ r1.y;
                    const uint32_t Y2 = TL(s2, 0, 0) ^ TL(s3, 1, 1) ^ TL(s0, 2, 2) ^ TL(s1, 3, 3) ^ r1.z;
                    const uint32_t Y3 = TL(s3, 0, 0) ^ TL(s0, 1, 1) ^ TL(s1, 2, 2) ^ TL(s2, 3, 3) ^ r1.w;
                    const uint32_t Z0 = TL(Y1, 1, 1) ^ TL(Y2, 2, 2) ^ TL(Y3, 3, 3) ^ r2.x;
                    const uint32_t Z1 = TL(Y1, 0, 0) ^ TL(Y2, 1, 1) ^ TL(Y3, 2, 2) ^ r2.y;
                    const uint32_t Z2 = TL(Y2, 0, 0) ^ TL(Y3, 1, 1) ^ TL(Y1, 3, 3) ^ r2.z;
                    const uint32_t Z3 = TL(Y3, 0, 0) ^ TL(Y1, 2, 2) ^ TL(Y2, 3, 3) ^ r2.w;
                    L.pre0[j] = make_uint4(X0, Z0, Z1, Z2);
                    L.pre1[j] = Z3;
                    L.pre2[j] = (uint8_t)(s3 >> 24);
                }
            }
            L.sa[j] = (uint16_t)sa;
            L.seq[j] = q32;
            L.info[j] = info;
            L.inoff[j] = inoff;
            atomicAdd(&L.bins[bin], 1u);
        }
        __syncthreads();
        if (warp == 0) {   // exclusive scan of the 32 bin counts -> bin cursors
            uint32_t cb = L.bins[lane], x = cb;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= (uint32_t)o) x += y;
            }
            L.bins[lane] = x - cb;
        }
        __syncthreads();
        for (uint32_t j = tid; j < cnt_pk; j += F_THREADS) {
            const uint32_t info = L.info[j];
            const uint32_t bin = (info & INFO_OK) ? hmac_bin(true, esp_C(info & 0x7ffu)) : NBINS - 1;
            L.perm[atomicAdd(&L.bins[bin], 1u)] = (uint16_t)j;
        }
        __syncthreads();
        uint32_t total_pairs = 0;
        for (uint32_t p0 = 0; p0 < cnt_pk; p0 += F_THREADS) {   // pair prefix, position order
            const uint32_t pp = p0 + tid;
            const uint32_t pj = (pp < cnt_pk) ? L.perm[pp] : 0u;
            const uint32_t info = (pp < cnt_pk) ? L.info[pj] : 0u;
            const uint32_t np = (info & INFO_OK) ? (esp_nblk(esp_C(info & 0x7ffu)) + 1u) >> 1 : 0u;
            uint32_t tot;
            const uint32_t ex = block_exclusive_scan(np, L.scr, &tot);
            if (pp < F_SUPER) L.ppref[pp] = total_pairs + ex;
            const uint32_t gsum = __reduce_add_sync(0xffffffffu, np);
            if (lane == 0 && (pp >> 5) < F_GROUPS) {
                L.gneed[pp >> 5] = gsum;
                if (gsum) mbar_init(&L.gbar[pp >> 5], gsum);
            }
            if (np) {   // chunk map: first position of every 32-pair chunk
                const uint32_t q0 = total_pairs + ex;
                for (uint32_t cc = (q0 + 31u) >> 5; (cc << 5) < q0 + np; cc++) H.chunkpos[cc] = (uint16_t)pp;
            }
            total_pairs += tot;
        }
        if (tid == 0) {
            L.ppref[cnt_pk] = total_pairs;
            L.aes_next = 0;
            L.hmac_next = 0;
        }
        __syncthreads();
        if (tr && tid == 0 && base == p_begin) tr[1] = gtimer();

        {
            // ---- 2+3. dynamic roles: AES pair-chunks and HMAC groups --------------
            const uint32_t n_chunks = (total_pairs + 31u) >> 5;
            const uint32_t n_groups = (cnt_pk + 31u) >> 5;
            uint32_t aes_left = 1;
            for (;;) {
                const uint32_t g = *reinterpret_cast<volatile uint32_t *>(&L.hmac_next);
                if (g < n_groups && (L.gneed[g] == 0 || mbar_test_parity0(&L.gbar[g]))) {
                    uint32_t won = 0;
                    if (lane == 0) won = atomicCAS(&L.hmac_next, g, g + 1u) == g;
                    if (__shfl_sync(0xffffffffu, won, 0)) {
                        if (tr && lane == 0) {
                            atomicMin(&tr[4], gtimer());
                            atomicMax(&tr[5], gtimer());
                        }
                        hmac_group(T, B, L, base, g, cnt_pk, lane);
                    }
                    continue;
                }
                if (aes_left) {
                    uint32_t cidx = 0;
                    if (lane == 0) cidx = atomicAdd(&L.aes_next, 1u);
                    cidx = __shfl_sync(0xffffffffu, cidx, 0);
                    if (cidx < n_chunks) {
                        aes_pair_chunk(B, L, H, lane4r, cidx, total_pairs, lane,
                                       (tr && blockIdx.x == 0 && cidx == 0) ? W.trace + 148 * 8 + 8 : nullptr);
                        continue;
                    }
                    aes_left = 0;
                    if (tr && lane == 0) atomicMax(&tr[2], gtimer());   // AES exhausted
                }
                if (g >= n_groups) break;           // everything claimed
                mbar_wait_parity0(&L.gbar[g]);      // sleep until group g is encrypted
            }
        }
        if (tr && lane == 0) atomicMax(&tr[3], gtimer());
        __syncthreads();   // shared metadata is reused by the next super-round
        if (tid < F_GROUPS && (tid << 5) < cnt_pk && L.gneed[tid]) mbar_inval(&L.gbar[tid]);
    }
    __syncthreads();
    if (tid < 4 && L.cnt[tid]) atomicAdd(&W.counters[tid], L.cnt[tid]);
    if (tid == 4 && blockIdx.x == 0) atomicAdd(&W.counters[4], 1ull);
}

int fused_grid(int num_sms) { return num_sms; }

uint32_t fused_ppc(uint32_t n, int grid)
{
    uint32_t ppc = (n + grid - 1) / grid;
    ppc = (ppc + 31u) & ~31u;
    return ppc < 32u ? 32u : ppc;
}

cudaError_t launch_fused(const DevTable &T, const DevWork &W, const BatchArgs &B, int grid,
                         cudaStream_t st)
{
    uint32_t ppc = fused_ppc(B.n, grid);
    uint32_t g = (B.n + ppc - 1) / ppc;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(g);
    cfg.blockDim = dim3(F_THREADS);
    cfg.dynamicSmemBytes = F_SMEM;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_fused, T, W, B, ppc);
}

cudaError_t setup_fused_attributes()
{
    return cudaFuncSetAttribute(k_fused, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)F_SMEM);
}

}  // namespace nba
