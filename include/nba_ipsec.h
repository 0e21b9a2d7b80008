/*
 * nba_ipsec.h -- C ABI of the B200-native IPsec ESP outbound hot path.
 *
 * What the library computes:
 *   NBA's "IPsec encryption gateway" offloads, per packet, "HMAC-SHA1 to
 *   authenticate the packets and AES-128CTR to encrypt them"
 *   (§4.1 "Sample applications"), using per-flow crypto
 *   contexts initialised once and reused "by only changing initial vector
 *   (IV) values".  The offloaded function consumes a
 *   *datablock*: byte ranges of packets given by offset/length (PAPER.md:329-343,
 *   §3.3 and Table 2) and returns whole packets with a size delta.  The
 *   framework validates fields before execution; invalid
 *   packets are dropped, not branched.
 *   The ESP wire format is not in the paper; it is fixed by the readings
 *   A1..A24 of DESIGN.md §3 (RFC 4303 tunnel mode, RFC 3686 AES-CTR,
 *   RFC 2404 HMAC-SHA1-96).  Per packet i with SA s = sa_idx[i] and inner
 *   IPv4 datagram P of D = in_len[i] bytes, the library writes at
 *   out_buf + out_off[i]:
 *       outer IPv4 (20 B) || SPI || seq || IV=BE64(seq) || AES-CTR(P||pad||p||4) || ICV(12 B)
 *   and out_len[i] = 48 + C, C = D + p + 2, p = (-(D+2)) mod 4.
 *
 * Threading/ordering: calls on one table must be serialised on one CUDA
 * stream (sequence numbers are stream-ordered state).  Different tables and
 * devices may run concurrently.
 *
 * Errors: argument errors are detected on the host before any work is
 * enqueued and return a negative NBA_IPSEC_E* code.  Per-packet problems are
 * NOT errors: the packet is dropped (out_len[i] = 0, pkts_dropped++) when
 * sa_idx[i] >= n_sa, D < 20, D > 1500, or the SA's 32-bit sequence number
 * space is exhausted (RFC 4303 §3.3.3).  Launch failures return
 * NBA_IPSEC_ECUDA; asynchronous faults surface at the caller's next
 * synchronisation.
 */
#ifndef NBA_IPSEC_H
#define NBA_IPSEC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
    NBA_IPSEC_OK = 0,
    NBA_IPSEC_EINVAL = -22,
    NBA_IPSEC_ENOMEM = -12,
    NBA_IPSEC_ENODEV = -19,
    NBA_IPSEC_ECUDA = -1000
};

#define NBA_IPSEC_MIN_DATAGRAM 20u    /* smallest inner IPv4 datagram (reading A15) */
#define NBA_IPSEC_MAX_DATAGRAM 1500u  /* largest inner datagram, PAPER.md:603 (A15) */
#define NBA_IPSEC_MAX_OVERHEAD 53u    /* 20 outer + 8 ESP + 8 IV + 3 pad + 2 trailer + 12 ICV */
#define NBA_IPSEC_MAX_SA       65536u /* per table */
#define NBA_IPSEC_MAX_BATCH    (1u << 22)

/* Per-SA parameters ("envelope contexts for all flows").
 * Integers are in host byte order. */
typedef struct {
    uint32_t spi;                    /* != 0 recommended (RFC 4303 §2.1); not checked */
    uint32_t tunnel_src, tunnel_dst; /* outer IPv4 addresses */
    uint8_t  aes_key[16];            /* AES-128 key (RFC 3686 §5 KEYMAT bytes 0..15) */
    uint8_t  ctr_nonce[4];           /* RFC 3686 nonce (KEYMAT bytes 16..19) */
    uint8_t  hmac_key[20];           /* RFC 2404: 160-bit HMAC-SHA1 key */
    uint32_t seq;                    /* last sequence number used; 0 => first packet gets 1 */
} nba_ipsec_sa_params;

typedef struct nba_ipsec_sa_table nba_ipsec_sa_table;  /* opaque; owns SA state + workspace */

/* One batch ("datablock" view).  For process_batch every
 * pointer is a DEVICE pointer on the table's device; for process_batch_host
 * every pointer is a HOST pointer (pinned memory recommended).
 *   in_buf  + in_off[i]  : inner IPv4 datagram i, in_len[i] bytes, any alignment
 *   sa_idx[i]            : SA index of packet i in [0, n_sa) (else dropped)
 *   out_buf + out_off[i] : output slot i; capacity must be >= in_len[i] + 53;
 *                          only bytes [0, out_len[i]) are written
 *   out_len[i]           : written: 48 + C, or 0 if dropped
 * in_buf and out_buf ranges must not overlap.  Slot i corresponds to packet i
 * (order preserved). */
typedef struct {
    const uint8_t  *in_buf;
    const uint32_t *in_off;
    const uint16_t *in_len;
    const uint32_t *sa_idx;
    uint8_t        *out_buf;
    const uint32_t *out_off;
    uint16_t       *out_len;
    uint32_t        n_pkts;
} nba_ipsec_batch;

/* Build the per-device SA table (AES-128 key schedules per FIPS-197 §5.2,
 * HMAC-SHA1 inner/outer midstates per RFC 2104) and a workspace sized for
 * max_batch_pkts packets.  `sas` is copied; the caller may free it on return.
 * All device memory is allocated here (none in process_batch).
 * Returns NBA_IPSEC_EINVAL for NULL sas/out, n_sa == 0 or > NBA_IPSEC_MAX_SA,
 * max_batch_pkts == 0 or > NBA_IPSEC_MAX_BATCH; NBA_IPSEC_ENODEV for a bad
 * device; NBA_IPSEC_ENOMEM if allocation fails. */
int nba_ipsec_create_sa_table(const nba_ipsec_sa_params *sas, uint32_t n_sa, int cuda_device,
                              uint32_t max_batch_pkts, nba_ipsec_sa_table **out);

/* Enqueue the whole ESP outbound path for one batch on `cuda_stream`
 * (a cudaStream_t; NULL = legacy default stream) and return immediately.
 * Device pointers only.  n_pkts == 0 is a no-op returning NBA_IPSEC_OK.
 * b->sa_idx may be NULL if a flow table is set (nba_ipsec_set_flow_table): the
 * packets' SAs are then looked up on the GPU first.
 * Returns NBA_IPSEC_EINVAL for NULL t/b, n_pkts > max_batch_pkts or a NULL
 * array with n_pkts > 0; NBA_IPSEC_ECUDA if a launch fails. */
int nba_ipsec_process_batch(nba_ipsec_sa_table *t, const nba_ipsec_batch *b, void *cuda_stream);

/* Same computation with HOST buffers (end-to-end path): copies
 * in_buf[0, in_buf_bytes) host->device, runs the path, copies
 * out_buf[0, out_buf_bytes) device->host.  The per-packet arrays (in_off,
 * in_len, sa_idx, out_off, out_len) are read / written by the kernels in place
 * when all five are page-locked memory the device can address (cudaHostAlloc,
 * cudaHostRegister), else staged with copies like in_buf.  The copies
 * and the kernels run on three internal streams with two staging slots, so
 * consecutive calls overlap batch k+1's copy-in and batch k-1's copy-out with
 * batch k's kernels (pinned host memory makes the copies asynchronous).
 * Ordering: the kernels start after all work already on `cuda_stream`, and
 * later work on `cuda_stream` waits for them (so the SA counters follow call
 * order, also when mixed with nba_ipsec_process_batch).  The OUTPUTS reach host
 * memory asynchronously: call nba_ipsec_host_wait(t, stream) and synchronise
 * that stream before reading out_buf / out_len or reusing any host buffer of
 * an earlier call.  out_buf[0, out_buf_bytes) is copied back whole: bytes
 * outside the slots' [0, out_len[i]) receive unspecified values.  Needs staging
 * reserved with nba_ipsec_reserve_host_io (EINVAL if it is too small). */
int nba_ipsec_process_batch_host(nba_ipsec_sa_table *t, const nba_ipsec_batch *b,
                                 uint64_t in_buf_bytes, uint64_t out_buf_bytes,
                                 void *cuda_stream);
/* Allocate (or grow) the two staging slots of the host path; synchronous. */
int nba_ipsec_reserve_host_io(nba_ipsec_sa_table *t, uint64_t in_buf_bytes,
                              uint64_t out_buf_bytes);
/* Make `cuda_stream` wait until every batch submitted so far through
 * nba_ipsec_process_batch_host has its outputs in host memory. */
int nba_ipsec_host_wait(nba_ipsec_sa_table *t, void *cuda_stream);

/* Free everything.  NULL -> NBA_IPSEC_OK.  Synchronises the table's device. */
int nba_ipsec_destroy(nba_ipsec_sa_table *t);

/* ---- auxiliary: tests, resume, bench -------------------------------------- */
typedef struct { uint64_t pkts_ok, pkts_dropped, bytes_in, bytes_out, batches; } nba_ipsec_counters;

/* Device counters accumulated since create.  Synchronises `cuda_stream`. */
int nba_ipsec_read_counters(nba_ipsec_sa_table *t, nba_ipsec_counters *out, void *cuda_stream);
/* Current per-SA sequence numbers (the only cross-batch state; re-import via
 * nba_ipsec_sa_params.seq for exact resume).  host_seq has n_sa entries.
 * Synchronises `cuda_stream`. */
int nba_ipsec_read_sa_seq(nba_ipsec_sa_table *t, uint32_t *host_seq, void *cuda_stream);
/* ---- batch rings: a fixed set of batch slots as one CUDA graph --------------
 *
 * A gateway that recycles a fixed pool of packet-buffer slots (PAPER.md:
 * 327-343: datablocks are byte ranges of the packets in their buffers) calls
 * the path on the same n_slots batches over and over.  ring_run enqueues
 * n_rounds passes over the slots, in slot order, on cuda_stream: the same
 * results as n_rounds x n_slots process_batch calls, without a host launch
 * per batch.  When every slot takes the one-kernel path (fused pipeline,
 * n_pkts <= 512 x SMs) a run is ONE persistent cooperative launch that walks
 * all its batches, keeping the AES tables in shared memory and letting a CTA
 * start the next batch while others finish -- by default software-pipelined
 * when every slot has SA indices and <= 448 packets per SM (the last two warps
 * of each CTA prepare the next batch's ranks and barrier arrival while the
 * others run this one; best for small packets), else plain
 * (nba_ipsec_ring_set_form switches; set NBA_IPSEC_RING_GRAPH before creation
 * to force the graph form); otherwise ring_create records process_batch for every slot
 * into a CUDA graph (the path keeps all per-batch state -- SA counters, the
 * one-kernel path's barrier base and batch epoch -- on the device, so the
 * recorded launches stay valid) and a run replays it n_rounds times.  The slots' DEVICE pointers and sizes are fixed at
 * creation (their contents may change between runs, in stream order).
 * The form and the pipeline are fixed when the ring is created.
 * NBA_IPSEC_EINVAL for NULL arguments, n_slots == 0 or > 4096, a slot that
 * process_batch would reject, or while profiling / tracing is enabled;
 * ring_run: NBA_IPSEC_EINVAL once the table's flow table was replaced
 * (nba_ipsec_set_flow_table) -- re-create the ring.  The ring must be
 * destroyed before its table. */
typedef struct nba_ipsec_ring nba_ipsec_ring;
int nba_ipsec_ring_create(nba_ipsec_sa_table *t, const nba_ipsec_batch *slots, uint32_t n_slots,
                          nba_ipsec_ring **out);
int nba_ipsec_ring_run(nba_ipsec_ring *r, uint32_t n_rounds, void *cuda_stream);
/* Exactly n_batches batches, slot after slot starting at the ring's cursor
 * (0 after creation), which then advances by n_batches mod n_slots: a run may
 * stop mid-rotation and the next one continues where it stopped.  Results are
 * those of the same sequence of process_batch (process_inbound) calls.
 * Persistent forms: ONE launch; graph form: whole rotations starting at slot 0
 * replay the graph, other batches are launched one by one.  ring_run(n) runs
 * n x n_slots batches from the cursor (which it leaves unchanged).
 * NBA_IPSEC_EINVAL as ring_run, or when timestamps are set with fewer than
 * n_batches + 1 entries; n_batches == 0 is a no-op. */
int nba_ipsec_ring_run_batches(nba_ipsec_ring *r, uint32_t n_batches, void *cuda_stream);
int nba_ipsec_ring_cursor(const nba_ipsec_ring *r);          /* slot of the next batch */
/* Per-batch device timestamps of later runs (persistent forms only): dev_ts is
 * a DEVICE buffer of cap u64 entries owned by the caller; each run zeroes
 * entries [0, n_batches] on its stream, then writes ts[0] = the run's start and
 * ts[1 + b] = the latest end, over the CTAs, of batch b's iteration (globaltimer
 * ns).  dev_ts == NULL switches it off.  NBA_IPSEC_EINVAL for a graph ring or
 * cap < 2. */
int nba_ipsec_ring_set_timestamps(nba_ipsec_ring *r, unsigned long long *dev_ts, uint32_t cap);
enum { NBA_IPSEC_RING_GRAPH = 0, NBA_IPSEC_RING_PERSISTENT = 1, NBA_IPSEC_RING_PIPELINED = 2,
       NBA_IPSEC_RING_FREE = 3, NBA_IPSEC_RING_ROLES = 4 };
/* The form a run takes (NBA_IPSEC_RING_*); set_form switches a persistent ring
 * between PERSISTENT, PIPELINED, FREE -- the pipelined form without the
 * end-of-batch CTA barrier: a lane warp that finished its run starts the next
 * batch while longer runs go on (mixed-length batches) -- and ROLES: CTA
 * roles instead of warp roles, a few "sequencer" CTAs run every batch's
 * prologue (validity, per-SA ranks over the whole batch, sequence numbers,
 * PAPER.md:389-395 / RFC 4303 §3.3.3) and write one record per packet, the
 * other CTAs encrypt as soon as a batch's records are out, with no grid-wide
 * synchronisation between batches on their side.  ROLES fits slots with SA
 * indices, <= 512 packets per encrypting CTA and <= 2048 SAs (its sequencer
 * count: 6 for packets of <= 114 bytes and for mixed lengths, else 4;
 * NBA_IPSEC_ROLES_P at creation overrides) and is the default form of rings
 * whose every slot holds packets of one length, at most 1010 bytes, and of
 * mixed-length rings of more than 4 slots (there each batch's packets are
 * sorted by length onto the encrypting warps; NBA_IPSEC_RING_ROLES=0/1 at
 * creation overrides).  NBA_IPSEC_EINVAL for
 * graph rings or slots a form does not fit.  All give identical results. */
int nba_ipsec_ring_form(const nba_ipsec_ring *r);
int nba_ipsec_ring_set_form(nba_ipsec_ring *r, int form);
int nba_ipsec_ring_destroy(nba_ipsec_ring *r);   /* NULL -> OK */

/* Overwrite the per-SA sequence numbers with host_seq[0..n_sa) (HOST memory):
 * the hand-over of an SA's counter when another device takes it over
 * (reading L7) or an exact resume.  Enqueued on `cuda_stream`
 * after earlier work; synchronises it (host_seq may be reused on return).
 * NBA_IPSEC_EINVAL for NULL arguments. */
int nba_ipsec_write_sa_seq(nba_ipsec_sa_table *t, const uint32_t *host_seq, void *cuda_stream);
const char *nba_ipsec_strerror(int code);

/* Pipeline selection (both produce identical bytes):
 *   NBA_IPSEC_PIPE_FUSED   : one fused prologue/gather/AES/HMAC/scatter kernel when
 *                            n_pkts <= 512 x SM count (cooperative launch, grid
 *                            barriers), else prologue kernel + fused kernel (default)
 *   NBA_IPSEC_PIPE_UNFUSED : prologue, gather, AES-CTR, HMAC-SHA1, scatter kernels */
enum { NBA_IPSEC_PIPE_FUSED = 0, NBA_IPSEC_PIPE_UNFUSED = 1 };
int nba_ipsec_set_pipeline(nba_ipsec_sa_table *t, int pipeline);
/* Number of kernel launches the most recent process_batch call enqueued
 * (2 before the first call). */
int nba_ipsec_launches_per_batch(nba_ipsec_sa_table *t);
/* Number of kernel launches the most recent process_inbound call enqueued:
 * 1 when n_pkts <= 512 x SM count (one cooperative kernel, the anti-replay
 * decision behind two grid barriers inside it), else 3 (3 before the first
 * call). */
int nba_ipsec_inbound_launches_per_batch(nba_ipsec_sa_table *t);

/* Per-kernel timing with CUDA events recorded on the caller's stream between
 * the kernels of each batch.  enable=1 starts (and resets) collection;
 * nba_ipsec_profile_read synchronises the device, and returns per-kernel sums
 * of milliseconds over all profiled batches (ms[k], k < *n_kernels, at most
 * max entries) with short kernel names (names[k] static strings), and the
 * number of profiled batches. */
int nba_ipsec_profile_enable(nba_ipsec_sa_table *t, int enable);
int nba_ipsec_profile_read(nba_ipsec_sa_table *t, double *ms, const char **names, int max,
                           int *n_kernels, uint32_t *n_batches);

/* Debug: per-CTA phase timestamps (%globaltimer ns) of the last fused batch,
 * 8 words per CTA: start, metadata done, AES done, HMAC done, first group
 * ready, last group ready.  Only when the table was created with the
 * environment variable NBA_IPSEC_TRACE set; otherwise NBA_IPSEC_EINVAL.
 * Synchronises the device. */
int nba_ipsec_debug_trace(nba_ipsec_sa_table *t, uint64_t *host, uint32_t n_words);

/* Host-only helpers exported for tests of the library's own setup code
 * (no device needed): the AES-128 key schedule (FIPS-197 §5.2; 44 words,
 * word i = bytes w[4i..4i+3] of the standard, big-endian) and the HMAC-SHA1
 * inner/outer chaining values after compressing K0^ipad / K0^opad
 * (RFC 2104 §2; FIPS 180-4 §6.1.2). */
void nba_ipsec_host_aes128_key_schedule(const uint8_t key[16], uint32_t w[44]);
void nba_ipsec_host_hmac_sha1_midstates(const uint8_t key[20], uint32_t hin[5], uint32_t hout[5]);

/* ---- flow -> SA lookup on the GPU --------------------------
 *
 * crypto contexts exist per flow and are set up at startup.  The
 * caller registers its flows -- exact inner IPv4 5-tuples -- and the SA each
 * one uses; the lookup then finds every packet's SA on the GPU (readings
 * F1..F4):
 *   key of the inner datagram P (D = in_len bytes): none unless P is IPv4 with
 *   20 <= 4*IHL <= D; else (src, dst, protocol, sport, dport), the ports being
 *   the 4 bytes after the IPv4 header for TCP (6) / UDP (17) when the fragment
 *   offset is 0 and D >= 4*IHL + 4, and 0 otherwise;
 *   sa_idx[i] = SA of the flow with that key, or NBA_IPSEC_NO_SA (no key / no
 *   match; the path drops such a packet like any sa_idx >= n_sa). */
#define NBA_IPSEC_NO_SA 0xffffffffu

typedef struct {
    uint32_t src, dst;       /* host order */
    uint16_t sport, dport;   /* 0 for portless protocols / non-first fragments */
    uint8_t  proto;
    uint8_t  pad_[3];
    uint32_t sa;             /* SA index, < n_sa */
} nba_ipsec_flow;

/* Build (replace) the device flow table from `flows` (copied; synchronous).
 * NBA_IPSEC_EINVAL for NULL flows with n_flows > 0, an sa >= n_sa, duplicate
 * keys, or n_flows > 2^26; NBA_IPSEC_ENOMEM if allocation fails.  n_flows = 0
 * removes the table. */
int nba_ipsec_set_flow_table(nba_ipsec_sa_table *t, const nba_ipsec_flow *flows, uint32_t n_flows);
/* Enqueue the lookup for n packets (DEVICE pointers) on `cuda_stream`:
 * sa_idx[i] <- the packet's SA or NBA_IPSEC_NO_SA.  NBA_IPSEC_EINVAL if no flow
 * table is set or n > max_batch_pkts.  nba_ipsec_process_batch also accepts
 * b->sa_idx == NULL when a flow table is set: it then runs this lookup first. */
int nba_ipsec_lookup_sa(nba_ipsec_sa_table *t, const uint8_t *in_buf, const uint32_t *in_off,
                        const uint16_t *in_len, uint32_t n_pkts, uint32_t *sa_idx,
                        void *cuda_stream);

/* ---- single-ingress redistribution ---------------
 *
 * With SA-hash sharding GPU g owns the SAs s with s mod world = g (local index
 * s / world).  When all traffic enters at one GPU, route_pack sorts a batch by
 * owner -- stable, so each owner receives its packets in batch order and the
 * per-SA sequence numbers are those of one sequential gateway -- and packs it
 * into destination-major send arrays for one all-to-all per array (NCCL over
 * NVLink; paper_conf_eurosys_kimjlmsm15_b200/redistribute.py):
 *   send_buf : packet bytes, destination 0's packets first, back to back
 *   send_len : their lengths; send_sa: their LOCAL SA indices (s / world)
 *   dest_counts[d], dest_bytes[d] (DEVICE, world + 1 entries): packets and
 *   bytes per destination; entry `world` counts packets with s >= n_sa_total,
 *   which are not sent.
 * All pointers are DEVICE pointers; sizes: send_buf >= the batch's bytes,
 * send_len / send_sa >= n_pkts entries, workspace >= route_workspace_bytes.
 * world must be 1..8.  Enqueued on `cuda_stream` (3 kernel launches). */
int nba_ipsec_route_workspace_bytes(uint32_t max_pkts, uint32_t world, uint64_t *bytes);
int nba_ipsec_route_pack(const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                         const uint32_t *sa_global, uint32_t n_pkts, uint32_t n_sa_total,
                         uint32_t world, void *workspace, uint8_t *send_buf, uint16_t *send_len,
                         uint32_t *send_sa, uint64_t *dest_counts, uint64_t *dest_bytes,
                         void *cuda_stream);
/* As nba_ipsec_route_pack with an explicit ownership map instead of s mod world
 * (the adaptive split below): sa_map (DEVICE, n_sa_total entries) holds
 * owner << 24 | local index for every SA, owner < world, local < 2^24; send_sa
 * receives the local index.  sa_map == NULL is route_pack.  A packet whose
 * map entry names an owner >= world is counted in dest_counts[world] and not
 * sent. */
int nba_ipsec_route_pack_map(const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                             const uint32_t *sa_global, uint32_t n_pkts, uint32_t n_sa_total,
                             const uint32_t *sa_map, uint32_t world, void *workspace,
                             uint8_t *send_buf, uint16_t *send_len, uint32_t *send_sa,
                             uint64_t *dest_counts, uint64_t *dest_bytes, void *cuda_stream);

/* Single-ingress dispatch straight into the owners' receive buffers: the
 * routing of route_pack_map (same destinations, same owner-local order) and
 * the data movement in one pass -- one warp per packet writes its bytes,
 * offset, length and local SA index into rx[owner], which may be this
 * device's memory or a peer GPU's mapped over NVLink (cudaIpcOpenMemHandle /
 * peer access), so no send buffer and no collective sit between routing and
 * the owners' process_batch.  rx: DEVICE array of `world` descriptors whose
 * pointers are valid on the calling device; receiver d gets its packets at
 * positions 0..count-1 (batch order), offsets into its buf, and
 * count[0] = packets, count[1] = bytes (written by the dispatch).  Each
 * receiver needs cap_pkts >= its packets and cap_bytes >= their bytes to take
 * all of them (cap_pkts = n_pkts and cap_bytes = the batch's bytes always do);
 * when its packets do not fit, the receiver gets the
 * longest prefix (in batch order) that fits both capacities, count[] says how
 * many packets / bytes that is, and nothing is written past the capacity --
 * the caller detects the overflow as dest_counts[d] > rx count (the dropped
 * suffix is the caller's to resend or count as lost).  Single ingress: one
 * dispatch per receive buffer at a time; the receivers may read them after the
 * caller's stream work completed (e.g. stream sync + a process-group barrier).
 * sa_map as in route_pack_map (NULL: owner = s mod world).  dest_counts /
 * dest_bytes (DEVICE, world + 1) as in route_pack.  4 kernel launches. */
typedef struct {
    uint8_t  *buf;          /* received packet bytes */
    uint32_t *off;          /* per packet: offset into buf */
    uint16_t *len;          /* per packet: length */
    uint32_t *sa;           /* per packet: local SA index */
    uint64_t *count;        /* [2]: packets, bytes */
} nba_ipsec_peer_rx;
int nba_ipsec_route_dispatch(const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                             const uint32_t *sa_global, uint32_t n_pkts, uint32_t n_sa_total,
                             const uint32_t *sa_map, uint32_t world, void *workspace,
                             const nba_ipsec_peer_rx *rx, uint64_t cap_pkts, uint64_t cap_bytes,
                             uint64_t *dest_counts, uint64_t *dest_bytes, void *cuda_stream);

/* ---- adaptive split of the SAs across devices -------------
 *
 * PAPER.md:351-365 (§3.4): NBA's load balancer hill-climbs the offloading
 * fraction w in [0%, 100%] by delta, choosing the direction "by observing if
 * throughput increases or decreases" (moving average of packets out per unit
 * time), waits for the workers to apply each update (2 .. 32 update intervals,
 * growing with w) and keeps perturbing w by delta.  Defaults: delta = 4%
 * (steps = 25), history 16384 samples, update interval 0.2 s.
 * Here w splits the SAs of a node of devices between its two halves (readings
 * L1..L7); host code only, no device work, no CUDA needed.
 *   observe(t_ns, dt_ns, pkts): one sample per completed batch -- the clock
 *   now, the batch's duration and the packets it transmitted; returns (in
 *   *step, may be NULL) the step k to apply, w = k / steps.  Deterministic:
 *   integer samples, exact comparisons.
 *   assign: owner[s] for s < n_sa under a binary tree of splits over n_dev <= 8
 *   devices: node i (heap order: root 0, children 2i+1, 2i+2) covering devices
 *   [lo, hi) and SAs [a, b) gives the last floor((b-a) * node_step[i] / steps)
 *   SAs to [lo + (hi-lo)/2, hi).  node_step has NBA_IPSEC_ALB_TREE_NODES
 *   entries (only internal nodes are read; may be NULL for n_dev = 1).
 *   sa_map (optional) receives owner << 24 | s: every device keeps all SAs, the
 *   owner's counter is the live one (nba_ipsec_write_sa_seq moves it). */
#define NBA_IPSEC_ALB_MAX_DEV 8u
#define NBA_IPSEC_ALB_TREE_NODES 15u

typedef struct {
    uint32_t steps;       /* K: w moves by 1/K (paper: delta = 4% -> 25); 1..10^6 */
    uint32_t init_step;   /* starting w = init_step / K; <= K */
    uint32_t history;     /* moving-average window, samples (paper: 16384); 1..2^26 */
    uint64_t update_ns;   /* observation interval (paper: 0.2 s); > 0 */
    uint32_t wait_min;    /* waiting interval at w = 0, in update intervals (paper: 2) */
    uint32_t wait_max;    /* ... at w = 100% (paper: 32); >= wait_min */
} nba_ipsec_alb_params;

typedef struct nba_ipsec_alb nba_ipsec_alb;   /* opaque controller */

void nba_ipsec_alb_default_params(nba_ipsec_alb_params *p);
/* NBA_IPSEC_EINVAL for NULL arguments or out-of-range parameters. */
int nba_ipsec_alb_create(const nba_ipsec_alb_params *p, nba_ipsec_alb **out);
int nba_ipsec_alb_observe(nba_ipsec_alb *a, uint64_t t_ns, uint64_t dt_ns, uint64_t pkts,
                          uint32_t *step);
/* Current step, direction (+1/-1) and number of updates so far (NULL: skip). */
int nba_ipsec_alb_state(const nba_ipsec_alb *a, uint32_t *step, int *direction, uint64_t *updates);
int nba_ipsec_alb_destroy(nba_ipsec_alb *a);   /* NULL -> OK */
/* NBA_IPSEC_EINVAL for n_dev outside 1..8, steps == 0, a node step > steps,
 * NULL owner (or NULL node_step with n_dev > 1), n_sa > 2^24. */
int nba_ipsec_alb_assign(uint32_t n_sa, uint32_t n_dev, const uint32_t *node_step, uint32_t steps,
                         uint32_t *owner, uint32_t *sa_map);

/* ---- ESP inbound: the mirror of the path ------------------
 *
 * RFC 4303 §3.4 receive processing in tunnel mode on the same SA table (the
 * SAs' keys; the receive state is separate from the outbound counter).  Per
 * packet i with s = sa_idx[i] and the outer IPv4 datagram of L = in_len[i]
 * bytes at in_buf + in_off[i] (readings B1..B9):
 *   1. s >= n_sa                                           -> DROP_SA
 *   2. format (§3.4.1-§3.4.2): 72 <= L <= 1552, C = L - 48 = 0 mod 4, version/IHL
 *      0x45, total length L, not a fragment, protocol 50, header checksum
 *      valid (RFC 1071), SPI = spi_s                       -> else DROP_FORMAT
 *   3. anti-replay (§3.4.3), window of NBA_IPSEC_REPLAY_WINDOW = 64 numbers:
 *      q = 0, q left of the window or already received     -> DROP_REPLAY
 *   4. ICV (§3.4.4.1): HMAC-SHA1-96 over SPI..ciphertext   -> else DROP_AUTH
 *   5. the window records q (only authenticated packets move it)
 *   6. decrypt (§3.4.4.2): AES-128-CTR, counter block nonce || IV (from the
 *      packet) || BE32(k+1) (RFC 3686)
 *   7. trailer: next header 4, pad bytes 1..p (§2.4), D = C - 2 - p >= 20
 *                                                          -> else DROP_TRAILER
 *   8. out_buf + out_off[i] <- the inner datagram (D bytes), out_len[i] = D.
 * The batch result equals processing the packets one by one in index order.
 * Window start (reading B6): an SA created with seq = s0 > 0 counts every
 * number <= s0 as received; s0 = 0 gives an empty window.
 * Slots: capacity >= in_len[i] - 48.  The library may write bytes [0, in_len[i]
 * - 48) of EVERY slot whose packet passes step 2 (decryption runs in parallel
 * with the ICV check, RFC 4303 §3.4.4.1); only [0, out_len[i]) is defined and
 * out_len[i] = 0 marks a dropped packet.  status (optional, may be NULL)
 * receives the NBA_IPSEC_IN_* code per packet. */
enum {
    NBA_IPSEC_IN_OK = 0,
    NBA_IPSEC_IN_DROP_SA = 1,
    NBA_IPSEC_IN_DROP_FORMAT = 2,
    NBA_IPSEC_IN_DROP_REPLAY = 3,
    NBA_IPSEC_IN_DROP_AUTH = 4,
    NBA_IPSEC_IN_DROP_TRAILER = 5
};
#define NBA_IPSEC_REPLAY_WINDOW 64u

typedef struct {
    const uint8_t  *in_buf;
    const uint32_t *in_off;
    const uint16_t *in_len;     /* outer datagram length L */
    const uint32_t *sa_idx;
    uint8_t        *out_buf;
    const uint32_t *out_off;
    uint16_t       *out_len;    /* written: D, or 0 if dropped */
    uint8_t        *status;     /* written if not NULL */
    uint32_t        n_pkts;
} nba_ipsec_in_batch;

typedef struct {
    uint64_t pkts_ok, drop_sa, drop_format, drop_replay, drop_auth, drop_trailer;
    uint64_t bytes_in, bytes_out, batches;
} nba_ipsec_in_counters;

/* Allocate the inbound state (receive windows initialised from the SAs' seq)
 * and workspace for max_batch_pkts packets.  Synchronous; idempotent.
 * NBA_IPSEC_ENOMEM if allocation fails. */
int nba_ipsec_enable_inbound(nba_ipsec_sa_table *t);
/* Enqueue ESP inbound for one batch (DEVICE pointers) on `cuda_stream`; three
 * kernel launches (decrypt+verify, replay scan, decide).  Same ordering rules
 * as process_batch.  NBA_IPSEC_EINVAL if inbound is not enabled, for NULL
 * arrays with n_pkts > 0 or n_pkts > max_batch_pkts. */
int nba_ipsec_process_inbound(nba_ipsec_sa_table *t, const nba_ipsec_in_batch *b, void *cuda_stream);
/* A batch ring (nba_ipsec_ring_create) of ESP inbound slots.  Form, chosen
 * at creation: when every slot has <= 448 packets per SM and every packet's
 * outer length is <= 640 B (read once from the slots' in_len, synchronously),
 * one software-pipelined persistent launch per run (the next batch's
 * metadata, the previous batch's replay row scans and decisions overlap the
 * current batch's crypto); otherwise process_inbound per slot recorded once
 * as a CUDA graph.  Environment overrides at creation:
 * NBA_IPSEC_RING_IN_PIPE=1 / =0 (pipelined whenever it fits / never),
 * NBA_IPSEC_RING_IN_PERSIST (a plain persistent launch per run),
 * NBA_IPSEC_RING_GRAPH (the graph).  Run / destroy with nba_ipsec_ring_run[_batches]
 * / nba_ipsec_ring_destroy.  Additionally NBA_IPSEC_EINVAL if inbound is not
 * enabled; NBA_IPSEC_ECUDA if reading the lengths fails. */
int nba_ipsec_ring_create_inbound(nba_ipsec_sa_table *t, const nba_ipsec_in_batch *slots,
                                  uint32_t n_slots, nba_ipsec_ring **out);
/* Enqueue (on `cuda_stream`) a reset of every receive window to its initial
 * state (reading B6), e.g. after re-keying; counters are kept. */
int nba_ipsec_reset_inbound(nba_ipsec_sa_table *t, void *cuda_stream);
/* Inbound counters since enable.  Synchronises `cuda_stream`. */
int nba_ipsec_read_in_counters(nba_ipsec_sa_table *t, nba_ipsec_in_counters *out, void *cuda_stream);
/* Receive windows: top[s] = highest authenticated number, bitmap[s] bit d set
 * iff number top[s] - d was received.  n_sa entries each.  Synchronises. */
int nba_ipsec_read_replay_window(nba_ipsec_sa_table *t, uint32_t *top, uint64_t *bitmap,
                                 void *cuda_stream);
/* As nba_ipsec_profile_read, for the inbound kernels (in_fused, in_replay, in_decide). */
int nba_ipsec_profile_read_inbound(nba_ipsec_sa_table *t, double *ms, const char **names, int max,
                                   int *n_kernels, uint32_t *n_batches);

#ifdef __cplusplus
}
#endif
#endif /* NBA_IPSEC_H */
