// internal.cuh -- device-side data layout and helpers shared by the kernels
// of libnba_ipsec.so (never by oracle/).  DESIGN.md §4 describes the layout.
#pragma once
#include <cstdint>

#include <vector_types.h>

#ifdef __CUDACC__
#include <cuda_runtime.h>

#include "nba_ipsec.h"
#endif

namespace nba {

constexpr uint32_t TILE = 1024;        // packets per scatter tile (unfused)
constexpr uint32_t PTILE = 256;        // packets per prologue / gather tile
constexpr uint32_t MIN_D = 20, MAX_D = 1500;
constexpr uint32_t MAX_REC_BYTES = 1536;  // roundup16(28 + 1504)
constexpr uint32_t DB_SLOT16 = 100;       // datablock uint4s per packet (>= fused slot of 1600 B)
constexpr uint32_t INVALID_SA = 0xffffffffu;
constexpr uint32_t INFO_OK = 0x80000000u;

// --- setup-time host arithmetic (host_tables.cpp) -------------------------
const uint32_t *host_te0();
const uint8_t *host_sbox();
void aes128_schedule_bytes(const uint8_t key[16], uint8_t rk[176]);
void hmac_midstates(const uint8_t key[20], uint32_t hin[5], uint32_t hout[5]);

// --- device SA table (a0) ---------------------------------------------------
// All words are little-endian images of the wire bytes unless noted.
struct DevTable {
    const uint4 *rk;        // [n_sa * 11] AES-128 round keys (FIPS-197 byte order)
    const uint4 *hmid;      // [n_sa * 3]  hin[0..4], hout[0..4] (SHA-1 words), 2 pad
    const uint4 *sahdr;     // [n_sa] {BE(spi), nonce bytes, BE(tun_src), BE(tun_dst)}
    uint32_t *seq;          // [n_sa] last sequence number used (mutable)
    uint32_t *seq_prev;     // [n_sa] value of seq before the current batch
    const uint32_t *te0;    // [256] T-table, row-0 byte in bits 0..7
    uint32_t n_sa;
    const uint4 *sal;       // [n_sa * SAL_U4] one 128-byte line per SA: AES key (round
                            //   key 0), sahdr, hmid[0..2], {hout[0..2], 0} -- what an
                            //   outbound lane loads, as three 256-bit loads (it
                            //   expands round keys 1..10 itself)
    const uint4 *timg;      // [8192] the 128 KB bank-replicated T-table image, laid out
                            //   exactly as in shared memory (bulk-copied per CTA)
};
constexpr uint32_t SAL_U4 = 8;   // uint4s per SA line (5 used)
constexpr uint32_t AES_TABLE_BYTES = 2u * 65536u;   // four 32x bank-replicated T-tables

// --- per-batch workspace ----------------------------------------------------
struct DevWork {
    uint32_t *lrank;        // [M]   within-tile per-SA rank
    uint32_t *m_rec;        // [M]   record offset in the datablock, 16-B units
    uint32_t *m_blk;        // [M+1] exclusive prefix of AES blocks (+ total)
    uint32_t *m_seq;        // [M]   ESP sequence number
    uint32_t *m_info;       // [M]   C | tos << 16 | INFO_OK  (0 = dropped / invalid)
    uint32_t *perm;         // [M]   HMAC processing order (length-binned)
    uint16_t *hist16;       // [n_sa][n_tiles] per-SA per-prologue-tile packet counts (SA-major;
                            //   all-zero between batches)
    uint32_t *hpfx;         // [n_sa][n_tiles] exclusive prefix of hist16 along each SA row
    unsigned long long *hbase;   // [n_sa][G] in-kernel prologue: epoch << 33 | (seq_prev + prefix)
    unsigned long long *pvote;   // [2][G] pipelined ring: epoch << 1 | "long batch" per CTA
    uint32_t *tile_rec;     // [max_tiles] record chunks per tile -> exclusive prefix
    uint32_t *tile_blk;     // [max_tiles] AES blocks per tile -> exclusive prefix
    uint32_t *tile_bin;     // [max_tiles * NBINS] HMAC length bins per tile -> prefix
    uint32_t *aes_start;    // [grid] first packet of each persistent AES / fused CTA
    uint32_t *ctl;          // [16] ticket, total_rec16, total_blk, ...
    unsigned long long *counters;  // [5] pkts_ok, pkts_dropped, bytes_in, bytes_out, batches
    unsigned long long *trace;     // [grid * 8 + 8] per-CTA phase timestamps (debug; may be null)
    uint32_t trace_pro;            // offset of the prologue's 8 trace words
    uint4 *db;              // datablock of ESP records (16-B aligned)
};

constexpr int CTL_TICKET = 0, CTL_TOTAL_REC = 1, CTL_TOTAL_BLK = 2, CTL_WORK = 3,
              CTL_BAR_COUNT = 4, CTL_BAR_GEN = 5, CTL_BAR_MONO = 6,
              // one-kernel fused path: arrivals before the current launch and the
              // last batch epoch, kept on the device so launches need no host
              // state (graph replay)
              CTL_BAR_BASE = 7, CTL_EPOCH = 8;
constexpr int NBINS = 32;   // HMAC bins by number of inner SHA-1 blocks (2..25)

struct BatchArgs {
    const uint8_t *in_buf;
    const uint32_t *in_off;
    const uint16_t *in_len;
    const uint32_t *sa_idx;       // null: the fused kernel looks the SAs up (flow table)
    uint8_t *out_buf;
    const uint32_t *out_off;
    uint16_t *out_len;
    uint32_t n;
    const uint4 *flow_table = nullptr;
    uint32_t flow_mask = 0;
};

// --- ESP inbound (readings B1..B9) ---------------
constexpr uint32_t IN_MIN_LEN = 48u + 24u;      // outer 20 + ESP 16 + C >= 24 + ICV 12
constexpr uint32_t IN_MAX_LEN = 48u + 1504u;
constexpr uint32_t IN_PIPE_MAX_LEN = 640u;   // inbound rings: pipelined form up to this outer length
constexpr uint32_t REPLAY_W = 64u;              // RFC 4303 §3.4.3 default window
// per-packet flags written by k_in_fused: bits 0..15 inner length D
constexpr uint32_t INF_FMT = 1u << 31, INF_ICV = 1u << 30, INF_TRL = 1u << 29;
enum : uint8_t { ST_OK = 0, ST_DROP_SA = 1, ST_DROP_FORMAT = 2, ST_DROP_REPLAY = 3,
                 ST_DROP_AUTH = 4, ST_DROP_TRAILER = 5 };
constexpr int N_IN_COUNTERS = 9;   // ok, 5 drop kinds, bytes_in, bytes_out, batches

struct InState {                    // per-SA receive windows + per-batch workspace
    uint32_t *top;                  // [n_sa] right edge (highest authenticated number)
    uint32_t *top_prev;             // [n_sa] before the current batch
    unsigned long long *bmp;        // [n_sa] bit d <-> number top - d
    unsigned long long *bmp_prev;   // [n_sa]
    uint32_t *flags;                // [M] INF_* | D
    uint32_t *seq;                  // [M] sequence number field
    uint32_t *lmax;                 // [M] max authenticated seq of the SA earlier in the tile
    uint32_t *hmax;                 // [n_sa][n_tiles] per-tile max (SA-major, zero between batches)
    uint32_t *pmx;                  // [n_sa][n_tiles] exclusive prefix max along each SA row
    unsigned long long *hkey;       // [hcap] (sa << 32 | seq) of authenticated packets
    uint32_t *hval;                 // [hcap] smallest packet index with that key
    unsigned long long *counters;   // [N_IN_COUNTERS]
    uint32_t *ctl;                  // [8] ticket, barrier count / generation
};

// The one-kernel inbound path's duplicate hashes by launch parity (the
// current one filled by the lanes, the next one cleared during the launch).
struct InHashPair {
    unsigned long long *hk[2];
    uint32_t *hv[2];
};

// The pipelined inbound ring's own buffers: duplicate hashes 1..3 (hash 0 is
// InState::hkey / hval), batch k's being hash k mod 4, and a scratch row of
// PIPE_MAX_PPC per-packet decision inputs per CTA (flags, sequence number,
// prefix max within the CTA, SA), written by batch k's tile part and read by
// its decisions during batch k + 1.
struct InPipeBufs {
    unsigned long long *hk1, *hk2, *hk3;
    uint32_t *hv1, *hv2, *hv3;
    uint4 *scr;                      // [G][448]
};

struct InBatchArgs {
    const uint8_t *in_buf;
    const uint32_t *in_off;
    const uint16_t *in_len;
    const uint32_t *sa_idx;
    uint8_t *out_buf;
    const uint32_t *out_off;
    uint16_t *out_len;
    uint8_t *status;                // may be null
    uint32_t n;
};

// --- flow -> SA lookup (readings F1..F4) ---------
// Open-addressing table, linear probing, capacity a power of two >= 2 x flows.
// Entry = {src, dst, sport << 16 | dport, proto | FLOW_VALID | sa << 16}.
constexpr uint32_t FLOW_VALID = 0x100u;
#if defined(__CUDACC__)
#define NBA_HD __host__ __device__
#else
#define NBA_HD
#endif
NBA_HD inline uint32_t flow_hash(uint32_t src, uint32_t dst, uint32_t ports, uint32_t proto)
{
    // murmur3-style finaliser over the folded key (host build and device probe)
    uint32_t h = src * 0x9E3779B1u;
    h ^= (dst << 13) | (dst >> 19);
    h = h * 0x85EBCA6Bu ^ ports;
    h = (h ^ (h >> 16)) * 0x7FEB352Du;
    h ^= proto * 0xC2B2AE35u;
    h = (h ^ (h >> 15)) * 0x846CA68Bu;
    return h ^ (h >> 16);
}

struct FlowArgs {
    const uint8_t *in_buf;
    const uint32_t *in_off;
    const uint16_t *in_len;
    uint32_t *sa_idx;
    uint32_t n;
};

#ifdef __CUDACC__
// --- launchers (one per kernel file) ----------------------------------------
cudaError_t launch_prologue(const DevTable &T, const DevWork &W, const BatchArgs &B,
                            uint32_t n_tiles, bool unfused, bool gridsync, cudaStream_t st);
cudaError_t launch_gather(const DevTable &T, const DevWork &W, const BatchArgs &B,
                          uint32_t n_tiles, uint32_t aes_grid, cudaStream_t st);
cudaError_t launch_aes(const DevTable &T, const DevWork &W, const BatchArgs &B, int grid,
                       cudaStream_t st);
cudaError_t launch_hmac(const DevTable &T, const DevWork &W, const BatchArgs &B,
                        cudaStream_t st);
cudaError_t launch_scatter(const DevTable &T, const DevWork &W, const BatchArgs &B,
                           uint32_t n_tiles, cudaStream_t st);
cudaError_t launch_fused(const DevTable &T, const DevWork &W, const BatchArgs &B, int grid,
                         bool merged, uint32_t *bar_base, uint32_t *epoch, cudaStream_t st);
bool fused_merged_ok(uint32_t n, int grid);
cudaError_t setup_prologue_attributes(uint32_t n_sa, uint32_t max_tiles, int num_sms, bool *gridsync);
cudaError_t setup_aes_attributes();
cudaError_t setup_fused_attributes();
// One run of a batch ring: batches first, first + 1, ... (mod n_slots) of the
// slot array, n_batches of them; ts (optional, zeroed by the host): ts[0] =
// run start, ts[1 + b] = max over CTAs of the global timer when batch b's
// iteration ended.
struct RingRun {
    uint32_t n_slots, first, n_batches;
    unsigned long long *ts;
};
cudaError_t launch_fused_ring_pipe(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                                   const RingRun &R, uint16_t *hist_b, int grid, cudaStream_t st);
cudaError_t launch_fused_ring_free(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                                   const RingRun &R, uint16_t *hist_b, int grid, cudaStream_t st);
bool fused_pipe_ok(uint32_t n, int grid);
// Role-split ring (k_fused_ring_roles): npro sequencer CTAs write one record
// per packet into a ring of ROLES_NREC record buffers, the other CTAs encrypt.
#ifndef NBA_ROLES_NREC
#define NBA_ROLES_NREC 4
#endif
constexpr uint32_t ROLES_NREC = NBA_ROLES_NREC;   // batches of records in flight
constexpr uint32_t ROLES_MAX_SA = 2048;     // per-warp SA counters in a sequencer's shared memory
constexpr uint32_t ROLES_RPP_MAX = 16416;   // packets per sequencer and batch (shared stash: 36 lane
                                            //   CTAs x 456 packets, a 65,536-packet batch at 4 sequencers)
constexpr uint32_t ROLES_CTL_WORDS = 2u * ROLES_NREC + 4u;   // ready[], consumed[], pbar, exit,
                                                             //   batch-0 bootstrap barrier / count
struct RolesBufs {
    uint32_t *ctl;      // [ROLES_CTL_WORDS] hand-off counters (zero between launches)
    uint32_t *rec;      // [ROLES_NREC][(grid - npro) * 512] per-packet sequence numbers (0: drop),
                        //   by packet index; sorted mode: uint4 {q, packet in the lane CTA's
                        //   range | D << 9 | SA << 20 (0xffffffff: none), in_off, out_off}
                        //   by lane slot
    uint32_t *cum;      // [(grid - npro) * 16] sorted mode: each lane warp's assigned work so far
    uint32_t sorted;    // 1: per-batch length-sorted lane slots (mixed-length rings)
    uint32_t stage;     // 1: sequencers stage SA indices / lengths by bulk copy (16-B aligned arrays)
    uint32_t boot;      // 1: every CTA numbers batch 0 (fixed-slot mode), the sequencers start at batch 1
    uint32_t *hist0;    // [n_sa][grid] bootstrap: per-(SA, CTA) counts -> exclusive prefixes over the CTAs
    uint32_t *tot0;     // [n_sa] bootstrap: the SA's valid packets in batch 0
    uint16_t *rows0;    // [grid][16][n_sa] bootstrap: per-warp SA group sizes of each CTA
    uint16_t *rank0;    // [grid * 512] bootstrap: each packet's rank among its CTA's packets of its SA
    uint32_t *ptot;     // [2][npro][n_sa] per-sequencer per-SA valid-packet totals
    uint8_t *scratch;   // [(grid - npro) * 256] output lines of the lanes' warm-up experiment
    uint32_t npro;      // sequencer CTAs
};
bool fused_roles_ok(uint32_t n, uint32_t n_sa, int grid, uint32_t npro);
cudaError_t launch_fused_ring_roles(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                                    const RingRun &R, const RolesBufs &Q, int grid, cudaStream_t st);
cudaError_t launch_fused_ring(const DevTable &T, const DevWork &W, const BatchArgs *slots,
                              const RingRun &R, uint16_t *hist_b, int grid, cudaStream_t st);
int aes_grid(int num_sms);
int fused_grid(int num_sms);
cudaError_t launch_in_fused(const DevTable &T, const InState &S, const InHashPair &HP,
                            const InBatchArgs &B, int grid, uint32_t hmask, uint32_t hfull,
                            bool merged, uint32_t *bar_base, cudaStream_t st);
bool in_merged_ok(uint32_t n, int grid);
cudaError_t launch_in_fused_ring(const DevTable &T, const InState &S, const InBatchArgs *slots,
                                 const RingRun &R, uint32_t hmask,
                                 unsigned long long *hkey_b, uint32_t *hval_b, int grid,
                                 cudaStream_t st);
cudaError_t launch_in_fused_ring_pipe(const DevTable &T, const InState &S, const InBatchArgs *slots,
                                      const RingRun &R, uint32_t hmask, const InPipeBufs &P, int grid,
                                      cudaStream_t st);
bool in_pipe_ok(uint32_t n, int grid);
cudaError_t launch_in_replay(const DevTable &T, const InState &S, const InBatchArgs &B,
                             uint32_t n_tiles, uint32_t hmask, bool gridsync, cudaStream_t st);
cudaError_t launch_in_decide(const DevTable &T, const InState &S, const InBatchArgs &B,
                             uint32_t n_tiles, uint32_t hmask, cudaStream_t st);
cudaError_t setup_inbound_attributes(uint32_t n_sa, uint32_t max_tiles, int num_sms, bool *gridsync);
cudaError_t launch_flow_lookup(const uint4 *table, uint32_t mask, const FlowArgs &A, cudaStream_t st);
size_t route_workspace_bytes(uint32_t max_pkts, uint32_t world);
cudaError_t launch_route(const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                         const uint32_t *sa, uint32_t n, uint32_t n_sa_total,
                         const uint32_t *sa_map, uint32_t world, void *ws, uint8_t *send_buf, uint16_t *send_len, uint32_t *send_sa,
                         unsigned long long *dest_counts, unsigned long long *dest_bytes,
                         cudaStream_t st, const nba_ipsec_peer_rx *rx = nullptr,
                         unsigned long long cap_pkts = 0, unsigned long long cap_bytes = 0);

// --- small device helpers ---------------------------------------------------
__device__ __forceinline__ uint32_t bswap32(uint32_t x) { return __byte_perm(x, 0, 0x0123); }

__device__ __forceinline__ unsigned long long gtimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ uint32_t lanemask_lt()
{
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// ESP sizes for an inner datagram of D bytes (A9):
// p = (-(D+2)) mod 4, C = D + p + 2, AES blocks ceil(C/16), record roundup16(28+C).
__device__ __forceinline__ uint32_t esp_pad(uint32_t D) { return (0u - (D + 2u)) & 3u; }
__device__ __forceinline__ uint32_t esp_C(uint32_t D) { return D + esp_pad(D) + 2u; }
__device__ __forceinline__ uint32_t esp_rec16(uint32_t C) { return (28u + C + 15u) >> 4; }
__device__ __forceinline__ uint32_t esp_nblk(uint32_t C) { return (C + 15u) >> 4; }
// inner SHA-1 blocks over (ipad block ||) SPI..trailer: message M = 16 + C bytes
// after the 64-byte key block; padded length (M + 9) rounded up to 64.
__device__ __forceinline__ uint32_t esp_nsha_inner(uint32_t C) { return (16u + C + 8u) / 64u + 1u; }
// HMAC length bin: longest first; invalid packets last.
__device__ __forceinline__ uint32_t hmac_bin(bool valid, uint32_t C)
{
    return valid ? (uint32_t)(NBINS - 1) - esp_nsha_inner(C) : (uint32_t)(NBINS - 1);
}

// 16 bytes starting at byte `sh` (0..15) of the 32-byte little-endian
// concatenation lo || hi.
__device__ __forceinline__ uint4 extract16(uint4 lo, uint4 hi, uint32_t sh)
{
    uint32_t q = sh >> 2, r = (sh & 3u) * 8u;
    uint32_t a0, a1, a2, a3, a4;
    switch (q) {
    case 0: a0 = lo.x; a1 = lo.y; a2 = lo.z; a3 = lo.w; a4 = hi.x; break;
    case 1: a0 = lo.y; a1 = lo.z; a2 = lo.w; a3 = hi.x; a4 = hi.y; break;
    case 2: a0 = lo.z; a1 = lo.w; a2 = hi.x; a3 = hi.y; a4 = hi.z; break;
    default: a0 = lo.w; a1 = hi.x; a2 = hi.y; a3 = hi.z; a4 = hi.w; break;
    }
    uint4 o;
    o.x = __funnelshift_r(a0, a1, r);
    o.y = __funnelshift_r(a1, a2, r);
    o.z = __funnelshift_r(a2, a3, r);
    o.w = __funnelshift_r(a3, a4, r);
    return o;
}

// 32 bytes (32-B aligned) in one 256-bit load (sm_100: LDG.E.ENL2.256)
__device__ __forceinline__ void ldg_nc_v8(const void *p, uint4 &a, uint4 &b)
{
    asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w), "=r"(b.x), "=r"(b.y), "=r"(b.z),
                   "=r"(b.w)
                 : "l"(p));
}

__device__ __forceinline__ uint4 ldg_nc_v4(const void *p)
{
    uint4 v;
    asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(p));
    return v;
}

__device__ __forceinline__ uint32_t get_byte(uint4 v, uint32_t j)
{
    uint32_t w = (j < 4) ? v.x : (j < 8) ? v.y : (j < 12) ? v.z : v.w;
    return (w >> ((j & 3u) * 8u)) & 0xffu;
}

__device__ __forceinline__ void set_byte(uint4 &v, uint32_t j, uint32_t b)
{
    uint32_t sh = (j & 3u) * 8u;
    uint32_t m = ~(0xffu << sh);
    if (j < 4) v.x = (v.x & m) | (b << sh);
    else if (j < 8) v.y = (v.y & m) | (b << sh);
    else if (j < 12) v.z = (v.z & m) | (b << sh);
    else v.w = (v.w & m) | (b << sh);
}

// Largest k in [0, n) with a[k] <= x, for non-decreasing a with a[0] <= x.
__device__ __forceinline__ uint32_t upper_bound_m1(const uint32_t *a, uint32_t n, uint32_t x)
{
    uint32_t lo = 0, len = n;
    while (len > 1) {
        uint32_t half = len >> 1;
        if (a[lo + half] <= x) lo += half;
        len -= half;
    }
    return lo;
}

// Block-wide exclusive scan of one u32 per thread (blockDim.x == 1024 or a
// multiple of 32 <= 1024).  `scratch` holds >= 32 u32.  Returns the exclusive
// prefix; *total receives the block sum.  Contains __syncthreads.
__device__ __forceinline__ uint32_t block_exclusive_scan(uint32_t v, uint32_t *scratch,
                                                         uint32_t *total)
{
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t nw = blockDim.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (uint32_t)o) x += y;
    }
    __syncthreads();
    if (lane == 31) scratch[warp] = x;
    __syncthreads();
    if (warp == 0) {
        uint32_t w = lane < nw ? scratch[lane] : 0u;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= (uint32_t)o) w += y;
        }
        scratch[lane] = w;   // inclusive warp-sum prefix
    }
    __syncthreads();
    uint32_t base = warp ? scratch[warp - 1] : 0u;
    *total = scratch[nw - 1];
    return base + x - v;
}

// Grid-wide barrier for a co-resident (cooperatively launched) grid: a
// monotonically increasing arrival counter; the host passes the count this
// barrier waits for (previous arrivals + gridDim.x), so it never needs a reset.
__device__ __forceinline__ void grid_sync_mono(uint32_t *count, uint32_t target)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(count, 1u);
        uint32_t v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(count) : "memory");
        } while ((int)(v - target) < 0);
        __threadfence();
    }
    __syncthreads();
}

// The same barrier in two halves, so a CTA can issue independent loads between
// its arrival and the wait: grid_arrive after a __syncthreads that orders the
// CTA's prior global writes; grid_wait ends with a __syncthreads.
#ifndef NBA_ARRIVE_RELEASE
#define NBA_ARRIVE_RELEASE 1
#endif
__device__ __forceinline__ void grid_arrive(uint32_t *count)
{
    if (threadIdx.x == 0) {
        if (NBA_ARRIVE_RELEASE) {
            // release RMW: orders the CTA's prior writes (made visible to this
            // thread by the preceding __syncthreads) before the arrival, without
            // the full fence's wait for everything in flight
            asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(count) : "memory");
        } else {
            __threadfence();
            atomicAdd(count, 1u);
        }
    }
}

#ifndef NBA_WAIT_FENCE
#define NBA_WAIT_FENCE 0
#endif
__device__ __forceinline__ void grid_wait(const uint32_t *count, uint32_t target)
{
    if (threadIdx.x == 0) {
        uint32_t v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(count) : "memory");
        } while ((int)(v - target) < 0);
        // the acquire load orders what follows; no trailing fence, which would
        // also wait for every load this thread still has in flight
        if (NBA_WAIT_FENCE) __threadfence();
    }
    __syncthreads();
}

// Exclusive prefix of the tile counts down SA column `sa` by one warp, then the
// SA counter advance (only the first (2^32-1 - seq) packets get numbers).
__device__ __forceinline__ void st_relaxed_u64(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// Where a row scan puts its exclusive prefixes: the prologue kernel writes
// hpfx[t] (read after a kernel boundary); the in-kernel prologue (BASE) writes
// hbase[t] = epoch << 33 | (seq_prev + prefix) with the batch's epoch, which the
// consuming CTA polls instead of waiting at a second grid barrier.
template <bool BASE>
__device__ __forceinline__ void put_prefix(const DevWork &W, size_t idx, uint32_t pfx, uint32_t old,
                                           uint32_t epoch)
{
    if (BASE)
        st_relaxed_u64(&W.hbase[idx], ((unsigned long long)epoch << 33) | ((unsigned long long)old + pfx));
    else
        W.hpfx[idx] = pfx;
}

// Exclusive prefix of the tile counts down SA row `sa` by one warp (coalesced:
// the matrix is SA-major), then the SA counter advance (only the first
// (2^32-1 - seq) packets get numbers).
template <bool BASE>
__device__ __forceinline__ void scan_sa_column(const DevTable &T, const DevWork &W, uint32_t sa,
                                               uint32_t n_tiles, uint32_t lane, uint32_t epoch,
                                               bool have_pre = false, uint32_t old_pre = 0)
{
    constexpr int U = 8;                       // 8 x 32 = 256 tiles per pass
    uint16_t *col = W.hist16 + (size_t)sa * n_tiles;
    const uint32_t old = have_pre ? old_pre : __shfl_sync(0xffffffffu, lane == 0 ? T.seq[sa] : 0u, 0);
    uint32_t carry = 0;
    for (uint32_t t0 = 0; t0 < n_tiles; t0 += 32u * U) {
        uint32_t h[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint32_t t = t0 + 32u * u + lane;
            h[u] = t < n_tiles ? __ldcg(&col[t]) : 0u;
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            if (t0 + 32u * u >= n_tiles) break;
            uint32_t x = h[u];
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= (uint32_t)o) x += y;
            }
            const uint32_t t = t0 + 32u * u + lane;
            if (t < n_tiles) {
                put_prefix<BASE>(W, (size_t)sa * n_tiles + t, carry + x - h[u], old, epoch);
                if (h[u]) col[t] = 0;            // re-arm for the next batch
            }
            carry += __shfl_sync(0xffffffffu, x, 31);
        }
    }
    if (lane == 0) {
        T.seq_prev[sa] = old;
        const uint32_t room = 0xffffffffu - old;
        T.seq[sa] = old + (carry < room ? carry : room);
    }
}

// The SA counter this warp's first row scan starts from (scan_all_columns with
// have_pre): T.seq of row `slot` (warp-per-row) or of row slot + lane * nslots
// (lane-per-row).  Only that scan writes T.seq of the row, so the value may be
// loaded early -- the merged kernel loads it before it waits at its barrier.
__device__ __forceinline__ uint32_t scan_first_old(const DevTable &T, uint32_t slot, uint32_t nslots,
                                                   uint32_t n_tiles, uint32_t lane)
{
    const size_t sa = n_tiles > 32u ? (size_t)slot : slot + (size_t)lane * nslots;
    return sa < T.n_sa ? T.seq[sa] : 0u;
}

// All SA rows, by `nslots` warps (this one is `slot`).  Long rows: one warp per
// SA (scan_sa_column).  Short rows (small batches, n_tiles <= 32): one LANE per
// SA, so a few warps still cover thousands of SAs in one memory round trip.
template <bool BASE = false>
__device__ __forceinline__ void scan_all_columns(const DevTable &T, const DevWork &W, uint32_t slot,
                                                 uint32_t nslots, uint32_t n_tiles, uint32_t lane,
                                                 uint32_t epoch = 0, bool have_pre = false,
                                                 uint32_t old_pre = 0)
{
    if (n_tiles > 32u) {
        for (uint32_t col = slot; col < T.n_sa; col += nslots)
            scan_sa_column<BASE>(T, W, col, n_tiles, lane, epoch, have_pre && col == slot, old_pre);
        return;
    }
    for (uint32_t k0 = 0; (size_t)k0 * nslots < T.n_sa; k0 += 32u) {
        // SA slot + k * nslots for k = k0 + lane: spread over all warps of the grid
        const size_t sa_l = slot + (size_t)(k0 + lane) * nslots;
        if (sa_l >= T.n_sa) continue;
        const uint32_t sa = (uint32_t)sa_l;
        uint16_t *col = W.hist16 + (size_t)sa * n_tiles;
        const uint32_t old = (have_pre && k0 == 0) ? old_pre : T.seq[sa];
        uint32_t h[32];
#pragma unroll
        for (uint32_t t = 0; t < 32u; t++) h[t] = t < n_tiles ? __ldcg(&col[t]) : 0u;
        uint32_t carry = 0;
#pragma unroll
        for (uint32_t t = 0; t < 32u; t++) {
            if (t < n_tiles) {
                put_prefix<BASE>(W, (size_t)sa * n_tiles + t, carry, old, epoch);
                if (h[t]) col[t] = 0;            // re-arm for the next batch
            }
            carry += h[t];
        }
        T.seq_prev[sa] = old;
        const uint32_t room = 0xffffffffu - old;
        T.seq[sa] = old + (carry < room ? carry : room);
    }
}

#endif

}  // namespace nba
