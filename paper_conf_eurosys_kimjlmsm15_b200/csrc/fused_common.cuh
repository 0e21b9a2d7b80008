// fused_common.cuh -- shared pieces of the lane-per-packet kernels (outbound
// k_fused.cu, inbound k_in_fused.cu): the shared-memory layout with the
// 64 KB-aligned bank-replicated T-tables, the PRMT-addressed table lookup, the
// RFC 3686 counter-block precompute and 4-block AES-128 step, and the
// destination-aligned output stream.
#pragma once
#ifndef NBA_STAGE_SERIAL
#define NBA_STAGE_SERIAL 0
#endif
#ifndef NBA_LPT               // 1: runs of 32 sorted packets to warps by LPT over sub-partitions
#define NBA_LPT 1
#endif
#ifndef NBA_SMSP_BALANCE      // 1: spread a super-round's packets over all 16 warps
#define NBA_SMSP_BALANCE 0
#endif
#include "aes_round.cuh"
#include "sha1.cuh"

namespace nba {

constexpr int F_THREADS = 512;            // 16 warps -> up to 128 registers
constexpr int F_SUPER = 512;              // packets per super-round (one per thread)

struct FusedLo {
    uint32_t sa[F_SUPER];          // by packet index in the super-round
    uint32_t info[F_SUPER];        // D | tos << 16 | INFO_OK  (0: dropped)
    uint32_t seq[F_SUPER];
    uint32_t inoff[F_SUPER];
    uint32_t outoff[F_SUPER];
    uint32_t aux0[F_SUPER];        // inbound: IV words of the packet
    uint32_t aux1[F_SUPER];
    uint16_t perm[F_SUPER];        // position -> packet index (length-sorted)
    uint4 rkA[4][F_THREADS];       // round keys 3..6 of the thread's current packet
    uint32_t bins[NBINS];
    unsigned long long cnt[4];
    uint32_t hkey[2 * F_SUPER];    // merged prologue: SA of each slot of the CTA's SA hash
    uint32_t hmask[2 * F_SUPER];   //   warps holding a group of that SA
    uint8_t wrun[F_THREADS / 32];  // warp -> run of 32 sorted positions (0xff: none)
    uint32_t pstat[3];             // pipelined ring: the next batch's AES steps (sum, max) and
                                   //   its "early round keys" decision
    unsigned long long tbar;       // mbarrier: the bulk copy of the T-table image landed
    uint32_t tailf[448];           // inbound pipelined ring: a batch's per-packet flags and
    uint32_t tailq[448];           //   sequence numbers and SA indices (by packet index) for
    uint32_t tails[448];           //   its replay tail
    uint32_t it0;                  // pipelined ring: this iteration's start (globaltimer, low word)
    uint32_t lanes_acc;            //   the lanes' latest end relative to it (this batch)
    uint32_t pro_delay;            //   the prologue warps' start delay for the next batch (ns)
    uint32_t stag_ns;              // pipelined ring: start delay of the upper lane warps
    uint32_t stag_acc;             //   (AES step 0 of the lower ones, measured per batch)
    uint32_t fr_ready;             // free-running ring: batches prepared (side -> lanes)
    uint32_t fr_taken;             //   lane warps' field takes so far (lanes -> side)
    uint32_t fr_load[16];          //   each lane warp's cumulative assigned cost
};

struct FusedHi {
    uint4 rkB[4][F_THREADS];       // round keys 7..10
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

// ---- T-table staging by bulk-async copy (TMA engine, cp.async.bulk) ---------
// The 128 KB bank-replicated table image is built once per SA table in global
// memory (DevTable::timg, exactly the shared-memory layout), and one thread
// per CTA copies it into shared memory with eight 16 KB cp.async.bulk
// operations that complete on an mbarrier (transaction count = 128 KB); the
// other threads go on with the batch's metadata / ranking and wait on the
// mbarrier only before their first table lookup.
#ifndef NBA_TMA_TABLES        // 0: the A/B baseline -- every thread copies the 1 KB T0 and
#define NBA_TMA_TABLES 1      //   stores the replicated / rotated image (aes_tables_to_smem)
#endif

__device__ __forceinline__ void tbar_init(unsigned long long *bar)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// One thread: arm the mbarrier for 128 KB and issue the copies.  Earlier
// generic-proxy accesses of the region (scratch use) are ordered before the
// async-proxy writes by the proxy fence (the caller has synchronised the CTA).
__device__ __forceinline__ void tables_bulk_issue(uint8_t *tabs, const uint4 *timg, unsigned long long *bar)
{
    const uint32_t b = smem_u32(bar), d = smem_u32(tabs);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "n"(AES_TABLE_BYTES)
                 : "memory");
#pragma unroll
    for (uint32_t i = 0; i < AES_TABLE_BYTES / 16384u; i++)
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 16384, [%2];"
                     ::"r"(d + 16384u * i), "l"(timg + 1024u * i), "r"(b)
                     : "memory");
}

// Start staging the tables (all threads call it; a CTA barrier must follow
// before the mbarrier is waited on).  init: first staging of this launch.
__device__ __forceinline__ void tables_stage(uint8_t *tabs, const DevTable &T, unsigned long long *bar,
                                             bool init)
{
    if (!NBA_TMA_TABLES) {
        aes_tables_to_smem(tabs, T.te0);
        return;
    }
    if (threadIdx.x == 0) {
        if (init) tbar_init(bar);
        tables_bulk_issue(tabs, T.timg, bar);
    }
}

// Wait until the phase with parity `phase` of the table mbarrier completed.
__device__ __forceinline__ void tables_bulk_wait(unsigned long long *bar, uint32_t phase)
{
    if (!NBA_TMA_TABLES) return;   // staged by plain stores before a CTA barrier
    const uint32_t b = smem_u32(bar);
    uint32_t ok;
    do {
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
                     "selp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok)
                     : "r"(b), "r"(phase)
                     : "memory");
    } while (!ok);
}

template <uint32_t OFF>
__device__ __forceinline__ uint32_t lds_abs(uint32_t a)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(a), "n"(OFF));
    return v;
}

// Warp-aggregated shared-memory counter increment: the lanes of a warp with
// the same key add together (one atomic per distinct key; 448 same-bin packets
// of a CTA otherwise serialise on one shared address), returning each lane's
// slot = old value + its rank among its peers.  All 32 lanes call it; lanes
// with active == false take no part.
__device__ __forceinline__ uint32_t warp_agg_add(uint32_t *ctr, uint32_t key, bool active)
{
    const uint32_t k = active ? key : 0xffffffffu;
    const uint32_t peers = __match_any_sync(0xffffffffu, k);
    const uint32_t leader = __ffs(peers) - 1;
    uint32_t lt;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
    uint32_t base = 0;
    if (active && (threadIdx.x & 31u) == leader) base = atomicAdd(&ctr[key], (uint32_t)__popc(peers));
    base = __shfl_sync(0xffffffffu, base, leader);
    return base + __popc(peers & lt);
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

__device__ __forceinline__ void prefetch_l2(const void *p)
{
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}

#ifndef NBA_BULK_PF            // 1: packet prefetches as bulk L2 prefetches of exactly the
#define NBA_BULK_PF 0         //   16-byte-aligned cover of the bytes used (else whole lines)
#endif

// L2 prefetch of bytes [p, p + n) of a packet (n > 0): one line prefetch at p,
// or (NBA_BULK_PF) a bulk prefetch of the 16-B aligned cover of the range
// (sectors only, no whole-line over-fetch of short packets).
__device__ __forceinline__ void prefetch_bytes(const uint8_t *p, uint32_t n)
{
    if (!NBA_BULK_PF) {
        prefetch_l2(p);
        return;
    }
    const uintptr_t a = reinterpret_cast<uintptr_t>(p), lo = a & ~(uintptr_t)15;
    const uint32_t sz = (uint32_t)(((a + n + 15u) & ~(uintptr_t)15) - lo);
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(lo), "r"(sz) : "memory");
}

__device__ __forceinline__ void stg_v4(void *p, uint32_t a, uint32_t b, uint32_t c, uint32_t d)
{
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(a), "r"(b), "r"(c), "r"(d)
                 : "memory");
}

// Bytes [lo, hi) of the 16-byte image (w0..w3) to chunk + [lo, hi); chunk 16-B aligned.
__device__ __forceinline__ void store_chunk_range(uint8_t *chunk, uint32_t w0, uint32_t w1,
                                                  uint32_t w2, uint32_t w3, uint32_t lo, uint32_t hi)
{
    if (lo == 0 && hi == 16) {
        stg_v4(chunk, w0, w1, w2, w3);
        return;
    }
    uint32_t x = lo;
    while (x < hi) {
        const uint32_t wi = x >> 2;
        const uint32_t w = wi == 0 ? w0 : wi == 1 ? w1 : wi == 2 ? w2 : w3;
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

// Streams the output packet (outer IPv4 || ESP header || ciphertext || ICV) as
// 32-bit words, in order, into destination-aligned 16-byte stores.  Output word
// w lands at byte e + 4w of the aligned chunk sequence starting at cp (e = the
// slot's misalignment); dest word k = funnel(out[k-q-1], out[k-q]) by r bits.
struct OutStream {
    uint8_t *cp;           // current 16-B aligned destination chunk
    uint32_t a0, a1, a2, a3;
    uint32_t p;            // next word position in the chunk (0..3)
    uint32_t prev;         // previous output word (for the funnel shift)
    uint32_t r;            // 8 * (e & 3)
    uint32_t lo;           // first byte of the current chunk that is ours

    __device__ __forceinline__ void init(uint8_t *dst)
    {
        const uintptr_t a = reinterpret_cast<uintptr_t>(dst);
        const uint32_t e = (uint32_t)(a & 15u);
        cp = reinterpret_cast<uint8_t *>(a - e);
        a0 = a1 = a2 = a3 = 0;
        p = e >> 2;
        prev = 0;
        r = (e & 3u) * 8u;
        lo = e;
    }
    __device__ __forceinline__ void place(uint32_t d)
    {
        a0 = p == 0 ? d : a0;
        a1 = p == 1 ? d : a1;
        a2 = p == 2 ? d : a2;
        a3 = p == 3 ? d : a3;
    }
    __device__ __forceinline__ void put(uint32_t v)
    {
        const uint32_t d = __funnelshift_l(prev, v, r);
        prev = v;
        place(d);
        if (++p == 4) {
            store_chunk_range(cp, a0, a1, a2, a3, lo, 16);
            cp += 16;
            p = 0;
            lo = 0;
        }
    }
    // 16 words whose dest words start at chunk position p (any): the whole
    // step without per-word selects.
    __device__ __forceinline__ void put16(const uint32_t (&v)[16])
    {
        uint32_t d[16];
#pragma unroll
        for (int i = 0; i < 16; i++) {
            d[i] = __funnelshift_l(i ? v[i - 1] : prev, v[i], r);
        }
        prev = v[15];
#define NBA_PUT16(P)                                                                             \
    {                                                                                            \
        uint32_t c[4] = {a0, a1, a2, a3};                                                        \
        _Pragma("unroll") for (int i = 0; i < 4 - (P); i++) c[(P) + i] = d[i];                   \
        store_chunk_range(cp, c[0], c[1], c[2], c[3], lo, 16);                                   \
        stg_v4(cp + 16, d[4 - (P)], d[5 - (P)], d[6 - (P)], d[7 - (P)]);                         \
        stg_v4(cp + 32, d[8 - (P)], d[9 - (P)], d[10 - (P)], d[11 - (P)]);                       \
        stg_v4(cp + 48, d[12 - (P)], d[13 - (P)], d[14 - (P)], d[15 - (P)]);                     \
        cp += 64;                                                                                \
        if ((P) > 0) a0 = d[16 - (P)];                                                           \
        if ((P) > 1) a1 = d[17 - (P)];                                                           \
        if ((P) > 2) a2 = d[18 - (P)];                                                           \
    }
        switch (p) {
        case 0: {
            // (lo != 0 only at the stream's start: bytes [0, lo) are not ours)
            store_chunk_range(cp, d[0], d[1], d[2], d[3], lo, 16);
            stg_v4(cp + 16, d[4], d[5], d[6], d[7]);
            stg_v4(cp + 32, d[8], d[9], d[10], d[11]);
            stg_v4(cp + 48, d[12], d[13], d[14], d[15]);
            cp += 64;
            break;
        }
        case 1: NBA_PUT16(1) break;
        case 2: NBA_PUT16(2) break;
        default: NBA_PUT16(3) break;
        }
#undef NBA_PUT16
        lo = 0;
    }
    // after the last word: the spill-over dest word (if r) and the final partial chunk
    __device__ __forceinline__ void finish(const uint8_t *end)
    {
        if (r) {
            place(__funnelshift_l(prev, 0u, r));
            if (++p == 4) {
                // the spill-over word completed a chunk: it ends inside it
                const uint32_t hi = (uint32_t)(end - cp);
                store_chunk_range(cp, a0, a1, a2, a3, lo, hi < 16u ? hi : 16u);
                cp += 16;
                p = 0;
                lo = 0;
                return;
            }
        }
        const intptr_t hi = end - cp;
        if (hi > 0) store_chunk_range(cp, a0, a1, a2, a3, lo, (uint32_t)hi);
    }
};


__device__ __forceinline__ void stg_v8(void *p, const uint32_t (&w)[8])
{
    asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(w[0]), "r"(w[1]),
                 "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7])
                 : "memory");
}

// Bytes [lo, hi) of the 32-byte image w[0..7] to chunk + [lo, hi); chunk 32-B aligned.
__device__ __forceinline__ void store_chunk32_range(uint8_t *chunk, const uint32_t (&w)[8], uint32_t lo,
                                                    uint32_t hi)
{
    if (lo == 0 && hi == 32) {
        stg_v8(chunk, w);
        return;
    }
    if (lo < 16) store_chunk_range(chunk, w[0], w[1], w[2], w[3], lo, hi < 16 ? hi : 16);
    if (hi > 16) store_chunk_range(chunk + 16, w[4], w[5], w[6], w[7], lo > 16 ? lo - 16 : 0, hi - 16);
}

// OutStream with 32-byte destination chunks (256-bit stores): a 64-byte step
// of ciphertext costs two store wavefronts per lane instead of four.
struct OutStream32 {
    uint8_t *cp;           // current 32-B aligned destination chunk
    uint32_t a[8];
    uint32_t p;            // next word position in the chunk (0..7)
    uint32_t prev;         // previous output word (for the funnel shift)
    uint32_t r;            // 8 * (e & 3)
    uint32_t lo;           // first byte of the current chunk that is ours

    __device__ __forceinline__ void init(uint8_t *dst)
    {
        const uintptr_t ad = reinterpret_cast<uintptr_t>(dst);
        const uint32_t e = (uint32_t)(ad & 31u);
        cp = reinterpret_cast<uint8_t *>(ad - e);
#pragma unroll
        for (int i = 0; i < 8; i++) a[i] = 0;
        p = e >> 2;
        prev = 0;
        r = (e & 3u) * 8u;
        lo = e;
    }
    __device__ __forceinline__ void place(uint32_t d)
    {
#pragma unroll
        for (int i = 0; i < 8; i++) a[i] = p == (uint32_t)i ? d : a[i];
    }
    __device__ __forceinline__ void put(uint32_t v)
    {
        const uint32_t d = __funnelshift_l(prev, v, r);
        prev = v;
        place(d);
        if (++p == 8) {
            store_chunk32_range(cp, a, lo, 32);
            cp += 32;
            p = 0;
            lo = 0;
        }
    }
    // 16 words whose dest words start at chunk position p (any)
    __device__ __forceinline__ void put16(const uint32_t (&v)[16])
    {
        uint32_t d[16];
#pragma unroll
        for (int i = 0; i < 16; i++) d[i] = __funnelshift_l(i ? v[i - 1] : prev, v[i], r);
        prev = v[15];
#define NBA_PUT16_32(P)                                                                        \
    {                                                                                          \
        uint32_t c[8];                                                                         \
        _Pragma("unroll") for (int i = 0; i < 8; i++) c[i] = i < (P) ? a[i] : d[i - (P)];      \
        store_chunk32_range(cp, c, lo, 32);                                                    \
        uint32_t c2[8];                                                                        \
        _Pragma("unroll") for (int i = 0; i < 8; i++) c2[i] = d[8 - (P) + i];                  \
        stg_v8(cp + 32, c2);                                                                   \
        cp += 64;                                                                              \
        _Pragma("unroll") for (int i = 0; i < (P); i++) a[i] = d[16 - (P) + i];               \
    }
        switch (p) {
        case 0: NBA_PUT16_32(0) break;
        case 1: NBA_PUT16_32(1) break;
        case 2: NBA_PUT16_32(2) break;
        case 3: NBA_PUT16_32(3) break;
        case 4: NBA_PUT16_32(4) break;
        case 5: NBA_PUT16_32(5) break;
        case 6: NBA_PUT16_32(6) break;
        default: NBA_PUT16_32(7) break;
        }
#undef NBA_PUT16_32
        lo = 0;
    }
    // after the last word: the spill-over dest word (if r) and the final partial chunk
    __device__ __forceinline__ void finish(const uint8_t *end)
    {
        if (r) {
            place(__funnelshift_l(prev, 0u, r));
            if (++p == 8) {
                const uint32_t hi = (uint32_t)(end - cp);
                store_chunk32_range(cp, a, lo, hi < 32u ? hi : 32u);
                return;
            }
        }
        const intptr_t hi = end - cp;
        if (hi > 0) store_chunk32_range(cp, a, lo, (uint32_t)hi);
    }
};

// ---- AES-128-CTR for one lane's packet (FIPS-197 §5.1 with T-tables) -------
// Counter block = n0 || iv0 || iv1 || BE32(k+1) (RFC 3686 §4; words are the
// little-endian loads of the wire bytes).  For k+1 < 256 only byte 15 varies,
// so round 1 is t0 = T3[R3 ^ (k+1)] ^ X0 (plus three row lookups of t0) and
// round 2 is u_c = T[row(t0)] ^ Z_c: rounds 1-2 are precomputed once per packet.
struct CtrPre {
    uint32_t X0, Z0, Z1, Z2, Z3, R3;
};

__device__ __forceinline__ CtrPre ctr_precompute(uint32_t lane4r, const uint4 &r0, const uint4 &r1,
                                                 const uint4 &r2, uint32_t n0, uint32_t iv0,
                                                 uint32_t iv1)
{
    const uint32_t s0 = n0 ^ r0.x, s1 = iv0 ^ r0.y, s2 = iv1 ^ r0.z, s3 = r0.w;
    CtrPre c;
    c.X0 = TL(s0, 0, 0) ^ TL(s1, 1, 1) ^ TL(s2, 2, 2) ^ r1.x;
    const uint32_t Y1 = TL(s1, 0, 0) ^ TL(s2, 1, 1) ^ TL(s3, 2, 2) ^ TL(s0, 3, 3) ^ r1.y;
    const uint32_t Y2 = TL(s2, 0, 0) ^ TL(s3, 1, 1) ^ TL(s0, 2, 2) ^ TL(s1, 3, 3) ^ r1.z;
    const uint32_t Y3 = TL(s3, 0, 0) ^ TL(s0, 1, 1) ^ TL(s1, 2, 2) ^ TL(s2, 3, 3) ^ r1.w;
    c.Z0 = TL(Y1, 1, 1) ^ TL(Y2, 2, 2) ^ TL(Y3, 3, 3) ^ r2.x;
    c.Z1 = TL(Y1, 0, 0) ^ TL(Y2, 1, 1) ^ TL(Y3, 2, 2) ^ r2.y;
    c.Z2 = TL(Y2, 0, 0) ^ TL(Y3, 1, 1) ^ TL(Y1, 3, 3) ^ r2.z;
    c.Z3 = TL(Y3, 0, 0) ^ TL(Y1, 2, 2) ^ TL(Y2, 3, 3) ^ r2.w;
    c.R3 = s3 >> 24;
    return c;
}

// Keystream of counter blocks 4 it + 1 .. 4 it + 4 (rounds 3..10; round keys
// 3..10 of this thread's packet staged in L.rkA / H.rkB), as 16 LE words.
// rkl / rkh: round keys 3..6 at rkl[(r - 3) * F_THREADS + slot], 7..10 at
// rkh[(r - 7) * F_THREADS + slot] (the thread's own slots in L.rkA / H.rkB, or
// other slots of the same arrays).
__device__ __forceinline__ void aes4_keystream(uint32_t lane4r, const CtrPre &c, uint32_t it,
                                               const uint4 *rkl, const uint4 *rkh, uint32_t slot,
                                               uint32_t (&ks)[16])
{
    uint32_t x[4][4];
#pragma unroll
    for (int b = 0; b < 4; b++) {
        const uint32_t t0 = TL((c.R3 ^ (4u * it + 1u + b)) << 24, 3, 3) ^ c.X0;
        x[b][0] = TL(t0, 0, 0) ^ c.Z0;
        x[b][1] = TL(t0, 3, 3) ^ c.Z1;
        x[b][2] = TL(t0, 2, 2) ^ c.Z2;
        x[b][3] = TL(t0, 1, 1) ^ c.Z3;
    }
#pragma unroll 1
    for (int r = 0; r < 7; r++) {
        const uint4 rk = r < 4 ? rkl[r * F_THREADS + slot] : rkh[(r - 4) * F_THREADS + slot];
#pragma unroll
        for (int b = 0; b < 4; b++) {
            const uint32_t u0 = TL(x[b][0], 0, 0) ^ TL(x[b][1], 1, 1) ^ TL(x[b][2], 2, 2) ^ TL(x[b][3], 3, 3) ^ rk.x;
            const uint32_t u1 = TL(x[b][1], 0, 0) ^ TL(x[b][2], 1, 1) ^ TL(x[b][3], 2, 2) ^ TL(x[b][0], 3, 3) ^ rk.y;
            const uint32_t u2 = TL(x[b][2], 0, 0) ^ TL(x[b][3], 1, 1) ^ TL(x[b][0], 2, 2) ^ TL(x[b][1], 3, 3) ^ rk.z;
            const uint32_t u3 = TL(x[b][3], 0, 0) ^ TL(x[b][0], 1, 1) ^ TL(x[b][1], 2, 2) ^ TL(x[b][2], 3, 3) ^ rk.w;
            x[b][0] = u0;
            x[b][1] = u1;
            x[b][2] = u2;
            x[b][3] = u3;
        }
    }
    const uint4 rk = rkh[3 * F_THREADS + slot];
#define NBA_FINAL(s0, s1, s2, s3)                                                               \
    ((TL(s0, 0, 2) & 0x000000ffu) | (TL(s1, 1, 3) & 0x0000ff00u) | (TL(s2, 2, 0) & 0x00ff0000u) | \
     (TL(s3, 3, 1) & 0xff000000u))
#pragma unroll
    for (int b = 0; b < 4; b++) {
        ks[4 * b + 0] = rk.x ^ NBA_FINAL(x[b][0], x[b][1], x[b][2], x[b][3]);
        ks[4 * b + 1] = rk.y ^ NBA_FINAL(x[b][1], x[b][2], x[b][3], x[b][0]);
        ks[4 * b + 2] = rk.z ^ NBA_FINAL(x[b][2], x[b][3], x[b][0], x[b][1]);
        ks[4 * b + 3] = rk.w ^ NBA_FINAL(x[b][3], x[b][0], x[b][1], x[b][2]);
    }
#undef NBA_FINAL
}

__device__ __forceinline__ void aes4_keystream(uint32_t lane4r, const CtrPre &c, uint32_t it,
                                               const FusedLo &L, const FusedHi &H, uint32_t tid,
                                               uint32_t (&ks)[16])
{
    aes4_keystream(lane4r, c, it, &L.rkA[0][0], &H.rkB[0][0], tid, ks);
}

// FIPS-197 §5.2 KeyExpansion of the lane's AES-128 key (round key 0 = r0) in
// registers, SubWord through the S-box bytes of the T-tables (the S-box value
// is byte 0 of T2[x], byte 1 of T3[x], byte 2 of T0[x], byte 3 of T1[x]);
// RotWord on a little-endian word image is a rotation by 8 bits, folded into
// which state byte indexes which table.  Round keys 1 and 2 are returned (the
// CTR precompute uses them), 3..10 go to L.rkA / H.rkB[.][tid].  40 lookups and
// ~100 ALU ops per packet replace 160 bytes of round-key loads per packet.
__device__ __forceinline__ void expand_key_slots(uint32_t lane4r, const uint4 &r0, uint4 &r1, uint4 &r2,
                                                 uint4 *rkl, uint4 *rkh, uint32_t slot)
{
    uint32_t w0 = r0.x, w1 = r0.y, w2 = r0.z, w3 = r0.w;
    uint32_t rc = 1u;
#pragma unroll
    for (int r = 1; r <= 10; r++) {
        const uint32_t t = (TL(w3, 1, 2) & 0x000000ffu) | (TL(w3, 2, 3) & 0x0000ff00u) |
                           (TL(w3, 3, 0) & 0x00ff0000u) | (TL(w3, 0, 1) & 0xff000000u);
        w0 ^= t ^ rc;                              // Rcon[r] = {rc, 0, 0, 0}
        w1 ^= w0;
        w2 ^= w1;
        w3 ^= w2;
        rc = ((rc << 1) ^ ((rc >> 7) * 0x11bu)) & 0xffu;   // xtime (constant per r)
        const uint4 k = make_uint4(w0, w1, w2, w3);
        if (r == 1) r1 = k;
        else if (r == 2) r2 = k;
        else if (r <= 6) rkl[(r - 3) * F_THREADS + slot] = k;
        else rkh[(r - 7) * F_THREADS + slot] = k;
    }
}

__device__ __forceinline__ void expand_key_lane(uint32_t lane4r, const uint4 &r0, uint4 &r1, uint4 &r2,
                                                FusedLo &L, FusedHi &H, uint32_t tid)
{
    expand_key_slots(lane4r, r0, r1, r2, &L.rkA[0][0], &H.rkB[0][0], tid);
}

// Round keys 3..10 of the lane's SA (FIPS-197 §5.2 schedule, built once per
// SA at setup, DevTable::rk) copied global -> the lane's own shared-memory
// slots L.rkA / H.rkB[.][tid] by cp.async (LDGSTS, 8 x 16 bytes, one commit
// group): issued before the batch's barrier wait / scans / polls, whose
// latency hides the copy; rk_async_wait() before the first AES round.  The
// lane's own copies only, so no CTA barrier is involved.
__device__ __forceinline__ void rk_async_issue(const uint4 *rk, uint32_t sa, FusedLo &L, FusedHi &H,
                                               uint32_t tid)
{
    const uint4 *src = rk + (size_t)sa * 11u + 3u;
#pragma unroll
    for (uint32_t r = 0; r < 8u; r++) {
        const uint32_t dst = r < 4u ? smem_u32(&L.rkA[r][tid]) : smem_u32(&H.rkB[r - 4u][tid]);
        asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src + r) : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

__device__ __forceinline__ void rk_async_wait()
{
    asm volatile("cp.async.wait_group 0;" ::: "memory");
}

// Warp-cooperative, coalesced staging of round keys 3..10 of each lane's SA
// (sa_me; INVALID_SA = none) into L.rkA / H.rkB: load m of the warp covers 128
// contiguous bytes of 4 lanes' SAs.  Followed by __syncwarp in the caller.
__device__ __forceinline__ void stage_round_keys(const uint4 *rk, FusedLo &L, FusedHi &H,
                                                 uint32_t sa_me, uint32_t warp, uint32_t lane)
{
#if NBA_STAGE_SERIAL
#pragma unroll
    for (int k = 0; k < 8; k++) {
        const uint32_t m = 32u * k + lane, owner = m >> 3, r = m & 7u;
        const uint32_t s = __shfl_sync(0xffffffffu, sa_me, owner);
        if (s != INVALID_SA) {
            const uint4 v = __ldg(&rk[(size_t)s * 11u + 3u + r]);
            const uint32_t slot = (warp << 5) + owner;
            if (r < 4) L.rkA[r][slot] = v;
            else H.rkB[r - 4][slot] = v;
        }
    }
    return;
#endif
    // all eight loads in flight before the first store
    uint4 v[8];
    uint32_t sv[8];
#pragma unroll
    for (int k = 0; k < 8; k++) {
        const uint32_t m = 32u * k + lane, owner = m >> 3, r = m & 7u;
        sv[k] = __shfl_sync(0xffffffffu, sa_me, owner);
        v[k] = sv[k] != INVALID_SA ? __ldg(&rk[(size_t)sv[k] * 11u + 3u + r]) : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int k = 0; k < 8; k++) {
        const uint32_t m = 32u * k + lane, owner = m >> 3, r = m & 7u;
        if (sv[k] != INVALID_SA) {
            const uint32_t slot = (warp << 5) + owner;
            if (r < 4) L.rkA[r][slot] = v[k];
            else H.rkB[r - 4][slot] = v[k];
        }
    }
}

// NW words of the byte stream at address a (any alignment); aligned 16-byte
// loads, none starting at or past `end`.
template <int NW>
__device__ __forceinline__ void load_words(uintptr_t a, uintptr_t end, uint32_t (&o)[NW])
{
    constexpr int NC = (4 * NW + 15) / 16 + 1;
    const uintptr_t ab = a & ~(uintptr_t)15;
    const uint32_t sh = (uint32_t)(a & 15u), rr = (sh & 3u) * 8u;
    uint32_t v[4 * NC];
#pragma unroll
    for (int i = 0; i < NC; i++) {
        const uintptr_t qa = ab + 16u * i;
        const uint4 c = qa < end ? ldg_nc_v4(reinterpret_cast<const void *>(qa)) : make_uint4(0, 0, 0, 0);
        v[4 * i] = c.x;
        v[4 * i + 1] = c.y;
        v[4 * i + 2] = c.z;
        v[4 * i + 3] = c.w;
    }
#define NBA_LW_CASE(Q)                                                                    \
    _Pragma("unroll") for (int w = 0; w < NW; w++) o[w] =                                 \
        __funnelshift_r(v[(Q) + w], v[(Q) + w + 1], rr);
    switch (sh >> 2) {
    case 0: NBA_LW_CASE(0) break;
    case 1: NBA_LW_CASE(1) break;
    case 2: NBA_LW_CASE(2) break;
    default: NBA_LW_CASE(3) break;
    }
#undef NBA_LW_CASE
}

// 16 words of the byte stream starting at address a (any alignment), in two
// halves so the loads can be in flight during the AES work: five aligned
// 16-byte loads (none starting at or past `end`), later the funnel shifts.
struct Raw5 {
    uint4 c[5];
    uint32_t sh;
};

__device__ __forceinline__ void load_raw5(uintptr_t a, uintptr_t end, Raw5 &r)
{
    const uintptr_t abase = a & ~(uintptr_t)15;
    r.sh = (uint32_t)(a & 15u);
    const uint4 z4 = make_uint4(0, 0, 0, 0);
#pragma unroll
    for (int i = 0; i < 5; i++) {
        const uintptr_t qa = abase + 16u * i;
        r.c[i] = qa < end ? ldg_nc_v4(reinterpret_cast<const void *>(qa)) : z4;
    }
}

// load_raw5 when all five 16-byte loads are known to be inside the stream
__device__ __forceinline__ void load_raw5_inb(uintptr_t a, Raw5 &r)
{
    const uintptr_t abase = a & ~(uintptr_t)15;
    r.sh = (uint32_t)(a & 15u);
#pragma unroll
    for (int i = 0; i < 5; i++) r.c[i] = ldg_nc_v4(reinterpret_cast<const void *>(abase + 16u * i));
}

__device__ __forceinline__ void extract16(const Raw5 &r, uint32_t (&o)[16])
{
    const uint32_t v[20] = {r.c[0].x, r.c[0].y, r.c[0].z, r.c[0].w, r.c[1].x, r.c[1].y, r.c[1].z,
                            r.c[1].w, r.c[2].x, r.c[2].y, r.c[2].z, r.c[2].w, r.c[3].x, r.c[3].y,
                            r.c[3].z, r.c[3].w, r.c[4].x, r.c[4].y, r.c[4].z, r.c[4].w};
    const uint32_t rr = (r.sh & 3u) * 8u;
#define NBA_PT_CASE(Q)                                                                    \
    _Pragma("unroll") for (int w = 0; w < 16; w++) o[w] =                                 \
        __funnelshift_r(v[(Q) + w], v[(Q) + w + 1], rr);
    switch (r.sh >> 2) {
    case 0: NBA_PT_CASE(0) break;
    case 1: NBA_PT_CASE(1) break;
    case 2: NBA_PT_CASE(2) break;
    default: NBA_PT_CASE(3) break;
    }
#undef NBA_PT_CASE
}

// The same with three 256-bit loads of the 32-byte aligned blocks covering
// [a, a + 64): fewer L1 data-pipe wavefronts per step (each lane's load touches
// its own line, so a warp-wide load costs one wavefront per lane whatever its
// width: 3 x 32 instead of 5 x 32).  Blocks starting at or past `end` are not
// read; a block that is read never crosses a 4 KB page, so it cannot fault
// where the datagram's own bytes do not.
struct Raw6 {
    uint4 c[6];
    uint32_t sh;
};

__device__ __forceinline__ void load_raw6(uintptr_t a, uintptr_t end, Raw6 &r)
{
    const uintptr_t abase = a & ~(uintptr_t)31;
    r.sh = (uint32_t)(a & 31u);
    const uint4 z4 = make_uint4(0, 0, 0, 0);
#pragma unroll
    for (int i = 0; i < 3; i++) {
        const uintptr_t qa = abase + 32u * i;
        if (qa < end) ldg_nc_v8(reinterpret_cast<const void *>(qa), r.c[2 * i], r.c[2 * i + 1]);
        else r.c[2 * i] = r.c[2 * i + 1] = z4;
    }
}

__device__ __forceinline__ void load_raw6_inb(uintptr_t a, Raw6 &r)
{
    const uintptr_t abase = a & ~(uintptr_t)31;
    r.sh = (uint32_t)(a & 31u);
#pragma unroll
    for (int i = 0; i < 3; i++)
        ldg_nc_v8(reinterpret_cast<const void *>(abase + 32u * i), r.c[2 * i], r.c[2 * i + 1]);
}

__device__ __forceinline__ void extract16(const Raw6 &r, uint32_t (&o)[16])
{
    uint32_t v[24];
#pragma unroll
    for (int i = 0; i < 6; i++) {
        v[4 * i] = r.c[i].x;
        v[4 * i + 1] = r.c[i].y;
        v[4 * i + 2] = r.c[i].z;
        v[4 * i + 3] = r.c[i].w;
    }
    const uint32_t rr = (r.sh & 3u) * 8u;
#define NBA_PT6_CASE(Q)                                                                   \
    _Pragma("unroll") for (int w = 0; w < 16; w++) o[w] =                                 \
        __funnelshift_r(v[(Q) + w], v[(Q) + w + 1], rr);
    switch (r.sh >> 2) {
    case 0: NBA_PT6_CASE(0) break;
    case 1: NBA_PT6_CASE(1) break;
    case 2: NBA_PT6_CASE(2) break;
    case 3: NBA_PT6_CASE(3) break;
    case 4: NBA_PT6_CASE(4) break;
    case 5: NBA_PT6_CASE(5) break;
    case 6: NBA_PT6_CASE(6) break;
    default: NBA_PT6_CASE(7) break;
    }
#undef NBA_PT6_CASE
}

// Counting sort of the super-round's packets by SHA-1 length (L.bins holds the
// counts; `bin` is thread j's packet's bin): L.perm[position] = packet.
__device__ __forceinline__ void length_sort(FusedLo &L, uint32_t j, uint32_t cnt_pk, uint32_t bin)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
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
    const uint32_t pos = warp_agg_add(L.bins, bin, j < cnt_pk);
    if (j < cnt_pk) L.perm[pos] = (uint16_t)j;
    __syncthreads();
    if (tid < NBINS) L.bins[tid] = 0;   // next round's counts (after its barrier)
    if (NBA_LPT && warp == 0) {
        // Runs of 32 sorted positions (one warp each) to warps: a warp costs
        // about its longest lane (all lanes step together), and warp w issues
        // on SM sub-partition w mod 4, so the runs go longest first to the
        // least loaded sub-partition (LPT).  Equal costs: run r -> warp r.
        constexpr uint32_t NW = F_THREADS / 32u;
        const uint32_t nruns = (cnt_pk + 31u) / 32u;
        uint32_t cost = 0;
        if (lane < nruns) {
            const uint32_t info = L.info[L.perm[32u * lane]];
            const uint32_t C = esp_C(info & 0x7ffu);
            cost = (info & INFO_OK) ? 8u * (esp_nsha_inner(C) + 1u) + 3u * ((C + 15u) >> 4) : 1u;
        }
        const uint32_t c0 = __shfl_sync(0xffffffffu, cost, 0);
        if (__all_sync(0xffffffffu, lane >= nruns || cost == c0)) {
            if (lane < NW) L.wrun[lane] = lane < nruns ? (uint8_t)lane : 0xffu;
        } else {
            // least-loaded sub-partition first, in registers (no local memory)
            uint32_t l0 = 0, l1 = 0, l2 = 0, l3 = 0, u0 = 0, u1 = 0, u2 = 0, u3 = 0, mine = 0xffu;
            constexpr uint32_t CAP = NW / 4u;
            for (uint32_t r = 0; r < nruns; r++) {
                const uint32_t cr = __shfl_sync(0xffffffffu, cost, r);
                uint32_t best = 0, bl = 0xffffffffu, bu = 0;
                if (u0 < CAP && l0 < bl) { best = 0; bl = l0; bu = u0; }
                if (u1 < CAP && l1 < bl) { best = 1; bl = l1; bu = u1; }
                if (u2 < CAP && l2 < bl) { best = 2; bl = l2; bu = u2; }
                if (u3 < CAP && l3 < bl) { best = 3; bl = l3; bu = u3; }
                if (lane == best + 4u * bu) mine = r;
                u0 += best == 0; u1 += best == 1; u2 += best == 2; u3 += best == 3;
                l0 += best == 0 ? cr : 0u; l1 += best == 1 ? cr : 0u;
                l2 += best == 2 ? cr : 0u; l3 += best == 3 ? cr : 0u;
            }
            if (lane < NW) L.wrun[lane] = (uint8_t)mine;
        }
    }
    if (NBA_LPT) __syncthreads();
}

// Lane -> position in the length-sorted order.  Default (NBA_LPT): warp w
// takes run L.wrun[w] (32 positions) as placed by length_sort.  Measured and
// kept off: NBA_SMSP_BALANCE, contiguous runs of ceil(cnt / 16) positions per
// warp so all 16 warps get packets (its warps finish together, yet 1514 B is
// 2% and 64 B 5% slower: the shared-memory / L1 data pipe is per SM, so the
// sub-partition imbalance it removes was not the bound).
__device__ __forceinline__ bool lane_position(const FusedLo &L, uint32_t cnt, uint32_t &pos)
{
    constexpr uint32_t NW = F_THREADS / 32u;
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    if (NBA_LPT) {
        const uint32_t r = L.wrun[warp];
        pos = 32u * r + lane;
        return r != 0xffu && pos < cnt;
    }
    if (!NBA_SMSP_BALANCE) {
        pos = threadIdx.x;
        return pos < cnt;
    }
    const uint32_t lw = (cnt + NW - 1u) / NW;
    pos = warp * lw + lane;
    return lane < lw && pos < cnt;
}

// ---- warp-specialised (software-pipelined) batch rings ---------------------
// Warps 0..13 ("lanes") carry a batch's packets, one per lane; warps 14..15
// ("prologue" / side warps) prepare the next batch meanwhile.
constexpr uint32_t PIPE_LANE_WARPS = 14;
constexpr uint32_t PIPE_MAX_PPC = PIPE_LANE_WARPS * 32u;          // 448 packets per CTA
constexpr uint32_t PIPE_P = F_THREADS - PIPE_MAX_PPC;             // 64 prologue threads

__device__ __forceinline__ void bar_sync_n(uint32_t id, uint32_t n)
{
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ void bar_arrive_n(uint32_t id, uint32_t n)
{
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}

// LPT placement of nruns runs (costs in lanes 0..nruns-1) onto the four SM
// sub-partitions (warp w issues on w mod 4; capq = lane warps on partition q):
// longest-first is the caller's order, each run goes to the least loaded
// partition with room (first minimum on ties), taking its next warp
// q + 4 * used_q.  Returns the run this lane's warp gets (0xff: none).  All
// state in registers (compare-select over the four partitions), so the
// prologue warps spill nothing.
__device__ __forceinline__ uint32_t lpt_place(uint32_t cost, uint32_t nruns, uint32_t lane,
                                              uint32_t cap0, uint32_t cap1, uint32_t cap2,
                                              uint32_t cap3)
{
    uint32_t l0 = 0, l1 = 0, l2 = 0, l3 = 0, u0 = 0, u1 = 0, u2 = 0, u3 = 0, mine = 0xffu;
    for (uint32_t r = 0; r < nruns; r++) {
        const uint32_t cr = __shfl_sync(0xffffffffu, cost, r);
        uint32_t best = 0, bl = 0xffffffffu, bu = 0;
        if (u0 < cap0 && l0 < bl) { best = 0; bl = l0; bu = u0; }
        if (u1 < cap1 && l1 < bl) { best = 1; bl = l1; bu = u1; }
        if (u2 < cap2 && l2 < bl) { best = 2; bl = l2; bu = u2; }
        if (u3 < cap3 && l3 < bl) { best = 3; bl = l3; bu = u3; }
        if (lane == best + 4u * bu) mine = r;
        u0 += best == 0; u1 += best == 1; u2 += best == 2; u3 += best == 3;
        l0 += best == 0 ? cr : 0u; l1 += best == 1 ? cr : 0u;
        l2 += best == 2 ? cr : 0u; l3 += best == 3 ? cr : 0u;
    }
    return mine;
}

// Flow -> SA lookup of one inner datagram P (D bytes), readings F1..F4: one
// unaligned 24-byte header load (two with IP options), then linear probing in
// the L2-resident open-addressing table.  INVALID_SA: no key or no match.
__device__ __forceinline__ uint32_t flow_lookup_one(const uint4 *__restrict__ table, uint32_t mask,
                                                    const uint8_t *P, uint32_t D)
{
    if (D < 20u) return INVALID_SA;
    const uintptr_t pa = reinterpret_cast<uintptr_t>(P);
    uint32_t w[6];
    load_words<6>(pa, pa + D, w);
    const uint32_t vihl = w[0] & 0xffu, ihl = vihl & 15u;
    if ((vihl >> 4) != 4u || ihl < 5u || D < 4u * ihl) return INVALID_SA;
    const uint32_t src = bswap32(w[3]), dst = bswap32(w[4]);
    const uint32_t proto = (w[2] >> 8) & 0xffu;
    const uint32_t frag = ((w[1] >> 8) & 0x1f00u) | (w[1] >> 24);   // bytes 6..7, 13 bits
    uint32_t ports = 0;
    if ((proto == 6u || proto == 17u) && frag == 0u && D >= 4u * ihl + 4u) {
        if (ihl == 5u) {
            ports = bswap32(w[5]);
        } else {
            uint32_t x[1];
            load_words<1>(pa + 4u * ihl, pa + D, x);
            ports = bswap32(x[0]);
        }
    }
    uint32_t h = flow_hash(src, dst, ports, proto) & mask;
    while (true) {
        const uint4 e = __ldg(&table[h]);
        if (!(e.w & FLOW_VALID)) return INVALID_SA;
        if (e.x == src && e.y == dst && e.z == ports && (e.w & 0xffu) == proto) return e.w >> 16;
        h = (h + 1u) & mask;
    }
}

}  // namespace nba
