// api.cu -- the C ABI of libnba_ipsec.so (include/nba_ipsec.h): SA-table
// construction (row a0), argument validation, workspace ownership and the
// per-batch launch sequence (rows a1..a5).
//
// per-flow crypto contexts are built once at startup and reused;
// the framework validates datablock fields before execution;
// offloads aggregate thousands of packets -- here a batch is up
// to max_batch_pkts packets that stay resident in HBM.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include "internal.cuh"
#include "nba_ipsec.h"

using namespace nba;

namespace {

constexpr int PROF_RING = 64;
constexpr int MAX_KERNELS = 8;

struct ProfSet {
    cudaEvent_t ev[MAX_KERNELS + 1] = {};
    int n_ev = 0;          // events recorded in this set (0 = empty)
    bool inbound = false;
    const char **names = nullptr;
};

}  // namespace

struct nba_ipsec_sa_table {
    int device = 0;
    uint32_t n_sa = 0, max_batch = 0, max_tiles = 0;
    int num_sms = 0;
    int grid_aes = 0, grid_fused = 0;
    int pipeline = NBA_IPSEC_PIPE_FUSED;
    bool gridsync = false;     // prologue phase 2 on all CTAs (grid barrier)
    bool allow_merged = true;  // prologue inside the fused kernel when the batch fits
    uint32_t bar_base = 0;     // arrivals so far at the fused kernel's grid barrier
    uint32_t epoch = 0;        // tag of the last in-kernel prologue's published bases
    int last_launches = 2;
    DevTable T{};
    DevWork W{};
    std::vector<void *> allocs;
    // host-I/O pipeline (process_batch_host): IO_DEPTH staging slots, copy-in /
    // compute / copy-out on three internal streams so batch k+1's H2D and batch
    // k-1's D2H overlap batch k's kernels
#ifndef NBA_IO_DEPTH
#define NBA_IO_DEPTH 2
#endif
    static constexpr int IO_DEPTH = NBA_IO_DEPTH;
    struct IoSlot {
        uint8_t *in = nullptr, *out = nullptr;
        uint32_t *meta = nullptr;   // in_off, sa_idx, out_off (u32) + in_len, out_len (u16)
        cudaEvent_t in_ready = nullptr, done = nullptr, out_done = nullptr;
    } io[IO_DEPTH];
    uint64_t io_in_bytes = 0, io_out_bytes = 0;
    bool io_ready = false;
    unsigned io_next = 0;
    cudaStream_t s_h2d = nullptr, s_comp = nullptr, s_d2h = nullptr;
    cudaEvent_t ev_call = nullptr;
    // profiling
    bool prof = false;
    ProfSet ring[PROF_RING];
    int ring_next = 0;
    uint32_t prof_batches = 0;
    double prof_ms[MAX_KERNELS] = {};
    int prof_nk = 0;
    const char **prof_names = nullptr;
    // ESP inbound (nba_ipsec_enable_inbound)
    std::vector<uint32_t> seq0;     // the SAs' initial seq (window start, reading B6)
    bool in_enabled = false, in_gridsync = false;
    uint32_t in_hcap = 0;
    InHashPair HP = {};           // the one-kernel inbound path's duplicate hashes
    uint32_t in_bar_base = 0;     // arrivals so far at the one-kernel inbound path's barriers
    uint32_t in_last_launches = 3;
    InState S{};
    uint32_t *in_top0 = nullptr;              // the windows' initial state (reset)
    unsigned long long *in_bmp0 = nullptr;
    double prof_in_ms[3] = {};
    uint32_t prof_in_batches = 0;
    // flow -> SA lookup (nba_ipsec_set_flow_table)
    uint4 *flow_table = nullptr;
    uint32_t flow_mask = 0;
    uint64_t flow_gen = 0;         // bumped by every nba_ipsec_set_flow_table
    uint32_t *flow_sa = nullptr;   // [max_batch] SA indices looked up for process_batch
};

namespace {

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev)
    {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard()
    {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

template <typename T>
cudaError_t dalloc(nba_ipsec_sa_table *t, T **p, size_t count)
{
    void *q = nullptr;
    cudaError_t e = cudaMalloc(&q, count * sizeof(T) + 256);
    if (e != cudaSuccess) return e;
    t->allocs.push_back(q);
    *p = static_cast<T *>(q);
    return cudaMemset(q, 0, count * sizeof(T) + 256);
}

void free_all(nba_ipsec_sa_table *t)
{
    for (void *p : t->allocs) cudaFree(p);
    t->allocs.clear();
    for (auto &s : t->ring)
        for (int k = 0; k < MAX_KERNELS + 1; k++)
            if (s.ev[k]) cudaEventDestroy(s.ev[k]);
}

const char *kernel_names_unfused[] = {"prologue", "gather", "aes_ctr", "hmac_sha1", "scatter"};
const char *kernel_names_fused[] = {"prologue", "fused"};
const char *kernel_names_merged[] = {"fused"};

void prof_drain_set(nba_ipsec_sa_table *t, ProfSet &s)
{
    if (s.n_ev == 0) return;
    cudaEventSynchronize(s.ev[s.n_ev - 1]);
    for (int k = 0; k + 1 < s.n_ev; k++) {
        float ms = 0.f;
        if (cudaEventElapsedTime(&ms, s.ev[k], s.ev[k + 1]) != cudaSuccess) continue;
        if (s.inbound) {
            if (k < 3) t->prof_in_ms[k] += ms;
        } else {
            t->prof_ms[k] += ms;
        }
    }
    if (s.inbound) {
        t->prof_in_batches++;
    } else {
        t->prof_nk = s.n_ev - 1;
        t->prof_names = s.names;
        t->prof_batches++;
    }
    s.n_ev = 0;
}

}  // namespace

extern "C" {

const char *nba_ipsec_strerror(int code)
{
    switch (code) {
    case NBA_IPSEC_OK: return "ok";
    case NBA_IPSEC_EINVAL: return "invalid argument";
    case NBA_IPSEC_ENOMEM: return "out of device memory";
    case NBA_IPSEC_ENODEV: return "no such CUDA device";
    case NBA_IPSEC_ECUDA: return "CUDA launch or runtime error";
    default: return "unknown error";
    }
}

int nba_ipsec_create_sa_table(const nba_ipsec_sa_params *sas, uint32_t n_sa, int cuda_device,
                              uint32_t max_batch_pkts, nba_ipsec_sa_table **out)
{
    if (!out) return NBA_IPSEC_EINVAL;
    *out = nullptr;
    if (!sas || n_sa == 0 || n_sa > NBA_IPSEC_MAX_SA || max_batch_pkts == 0 ||
        max_batch_pkts > NBA_IPSEC_MAX_BATCH)
        return NBA_IPSEC_EINVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || cuda_device < 0 || cuda_device >= ndev) {
        cudaGetLastError();
        return NBA_IPSEC_ENODEV;
    }
    DeviceGuard g(cuda_device);
    auto *t = new (std::nothrow) nba_ipsec_sa_table();
    if (!t) return NBA_IPSEC_ENOMEM;
    t->device = cuda_device;
    t->n_sa = n_sa;
    t->max_batch = max_batch_pkts;
    t->max_tiles = (max_batch_pkts + PTILE - 1) / PTILE;
    cudaDeviceGetAttribute(&t->num_sms, cudaDevAttrMultiProcessorCount, cuda_device);
    t->grid_aes = aes_grid(t->num_sms);
    t->grid_fused = t->grid_aes;

    // ---- a0: host-side key schedules, midstates, header words -------------
    std::vector<uint4> rk((size_t)n_sa * 11), hm((size_t)n_sa * 3), hdr(n_sa);
    std::vector<uint32_t> seq(n_sa);
    std::vector<uint4> sal((size_t)n_sa * SAL_U4, make_uint4(0, 0, 0, 0));
    for (uint32_t s = 0; s < n_sa; s++) {
        const nba_ipsec_sa_params &p = sas[s];
        uint8_t bytes[176];
        aes128_schedule_bytes(p.aes_key, bytes);
        std::memcpy(&rk[(size_t)s * 11], bytes, 176);
        uint32_t hin[5], hout[5];
        hmac_midstates(p.hmac_key, hin, hout);
        hm[(size_t)s * 3 + 0] = make_uint4(hin[0], hin[1], hin[2], hin[3]);
        hm[(size_t)s * 3 + 1] = make_uint4(hin[4], hout[0], hout[1], hout[2]);
        hm[(size_t)s * 3 + 2] = make_uint4(hout[3], hout[4], 0u, 0u);
        auto be_img = [](uint32_t v) {   // little-endian image of BE32(v)
            return ((v >> 24) & 0xffu) | ((v >> 8) & 0xff00u) | ((v << 8) & 0xff0000u) |
                   (v << 24);
        };
        uint32_t nonce;
        std::memcpy(&nonce, p.ctr_nonce, 4);
        hdr[s] = make_uint4(be_img(p.spi), nonce, be_img(p.tunnel_src), be_img(p.tunnel_dst));
        seq[s] = p.seq;
        uint4 *line = &sal[(size_t)s * SAL_U4];
        line[0] = rk[(size_t)s * 11];
        line[1] = hdr[s];
        line[2] = hm[(size_t)s * 3 + 0];
        line[3] = hm[(size_t)s * 3 + 1];
        line[4] = hm[(size_t)s * 3 + 2];
        line[5] = make_uint4(hout[0], hout[1], hout[2], 0u);   // words 4..5 = hout[3,4,-,-,0,1,2]
        line[6] = rk[(size_t)s * 11 + 1];                        // round keys 1, 2 (CTR precompute)
        line[7] = rk[(size_t)s * 11 + 2];
    }
    t->seq0 = seq;

    uint4 *d_rk = nullptr, *d_hm = nullptr, *d_hdr = nullptr, *d_sal = nullptr;
    uint32_t *d_seq = nullptr, *d_seq_prev = nullptr, *d_te0 = nullptr;
    uint4 *d_timg = nullptr;
    const uint32_t M = max_batch_pkts;
    cudaError_t e = cudaSuccess;
    auto chk = [&](cudaError_t x) {
        if (e == cudaSuccess && x != cudaSuccess) e = x;
    };
    chk(dalloc(t, &d_rk, rk.size()));
    chk(dalloc(t, &d_hm, hm.size()));
    chk(dalloc(t, &d_hdr, hdr.size()));
    chk(dalloc(t, &d_sal, sal.size()));
    chk(dalloc(t, &d_seq, n_sa));
    chk(dalloc(t, &d_seq_prev, n_sa));
    chk(dalloc(t, &d_te0, 256));
    chk(dalloc(t, &d_timg, AES_TABLE_BYTES / sizeof(uint4)));
    DevWork &W = t->W;
    chk(dalloc(t, &W.lrank, M));
    chk(dalloc(t, &W.m_rec, M));
    chk(dalloc(t, &W.m_blk, M + 1));
    chk(dalloc(t, &W.m_seq, M));
    chk(dalloc(t, &W.m_info, M));
    chk(dalloc(t, &W.perm, M));
    // columns: prologue tiles, or the fused kernel's CTAs when it runs the prologue
    const size_t cols = std::max<size_t>(t->max_tiles, (size_t)t->grid_fused);
    chk(dalloc(t, &W.hist16, cols * n_sa));
    chk(dalloc(t, &W.hpfx, cols * n_sa));
    chk(dalloc(t, &W.hbase, (size_t)t->grid_fused * n_sa));
    chk(dalloc(t, &W.pvote, 2ull * t->grid_fused));
    chk(dalloc(t, &W.tile_rec, t->max_tiles));
    chk(dalloc(t, &W.tile_blk, t->max_tiles));
    chk(dalloc(t, &W.tile_bin, (size_t)t->max_tiles * NBINS));
    chk(dalloc(t, &W.aes_start, (size_t)std::max(t->grid_aes, t->grid_fused)));
    chk(dalloc(t, &W.ctl, 16));
    chk(dalloc(t, &W.counters, 8));
    chk(dalloc(t, &W.db, (size_t)M * DB_SLOT16 + 16));
    if (std::getenv("NBA_IPSEC_TRACE")) chk(dalloc(t, &W.trace, (size_t)t->grid_fused * 8 + 64));
    W.trace_pro = (uint32_t)t->grid_fused * 8;
    if (e == cudaSuccess) {
        chk(cudaMemcpy(d_rk, rk.data(), rk.size() * sizeof(uint4), cudaMemcpyHostToDevice));
        chk(cudaMemcpy(d_hm, hm.data(), hm.size() * sizeof(uint4), cudaMemcpyHostToDevice));
        chk(cudaMemcpy(d_hdr, hdr.data(), hdr.size() * sizeof(uint4), cudaMemcpyHostToDevice));
        chk(cudaMemcpy(d_sal, sal.data(), sal.size() * sizeof(uint4), cudaMemcpyHostToDevice));
        chk(cudaMemcpy(d_seq, seq.data(), n_sa * sizeof(uint32_t), cudaMemcpyHostToDevice));
        chk(cudaMemcpy(d_te0, host_te0(), 256 * sizeof(uint32_t), cudaMemcpyHostToDevice));
        // the kernels' shared-memory table image (bulk-copied per CTA): entry x
        // of table j (Tj = rotl(T0, 8j)) at byte (j >> 1) * 64 KB + 256 x +
        // 128 (j & 1) + 4 lane, replicated over the 32 lanes (fused_common.cuh TL)
        std::vector<uint32_t> img(AES_TABLE_BYTES / 4);
        const uint32_t *te0 = host_te0();
        for (uint32_t j = 0; j < 4; j++)
            for (uint32_t x = 0; x < 256; x++) {
                const uint32_t v = j ? (te0[x] << (8 * j)) | (te0[x] >> (32 - 8 * j)) : te0[x];
                for (uint32_t l = 0; l < 32; l++)
                    img[(j >> 1) * 16384u + x * 64u + (j & 1u) * 32u + l] = v;
            }
        chk(cudaMemcpy(d_timg, img.data(), AES_TABLE_BYTES, cudaMemcpyHostToDevice));
    }
    if (e == cudaSuccess) chk(setup_prologue_attributes(n_sa, t->max_tiles, t->num_sms, &t->gridsync));
    // testing: force the last-CTA (non co-resident) fallback of the per-SA scans
    if (std::getenv("NBA_IPSEC_NO_GRIDSYNC")) t->gridsync = false;
    // testing: always use the separate prologue kernel
    if (std::getenv("NBA_IPSEC_NO_MERGE")) t->allow_merged = false;
    if (e == cudaSuccess) chk(setup_aes_attributes());
    if (e == cudaSuccess) chk(setup_fused_attributes());
    if (e == cudaSuccess) chk(cudaDeviceSynchronize());
    if (e != cudaSuccess) {
        cudaGetLastError();
        free_all(t);
        delete t;
        return e == cudaErrorMemoryAllocation ? NBA_IPSEC_ENOMEM : NBA_IPSEC_ECUDA;
    }
    t->T = DevTable{d_rk, d_hm, d_hdr, d_seq, d_seq_prev, d_te0, n_sa, d_sal, d_timg};
    *out = t;
    return NBA_IPSEC_OK;
}

static int enqueue(nba_ipsec_sa_table *t, const BatchArgs &B, cudaStream_t st)
{
    const uint32_t n_tiles = (B.n + PTILE - 1) / PTILE;      // prologue / gather tiles
    const uint32_t n_stiles = (B.n + TILE - 1) / TILE;       // scatter tiles
    ProfSet *ps = nullptr;
    if (t->prof) {
        ps = &t->ring[t->ring_next];
        prof_drain_set(t, *ps);        // only blocks if the ring wrapped
        t->ring_next = (t->ring_next + 1) % PROF_RING;
        for (int k = 0; k < MAX_KERNELS + 1; k++)
            if (!ps->ev[k]) cudaEventCreate(&ps->ev[k]);
        ps->n_ev = 0;
        ps->inbound = false;
    }
    auto mark = [&]() {
        if (ps) cudaEventRecord(ps->ev[ps->n_ev++], st);
    };
    const bool unfused = t->pipeline == NBA_IPSEC_PIPE_UNFUSED;
    const bool merged = !unfused && t->allow_merged && fused_merged_ok(B.n, t->grid_fused);
    if (ps) ps->names = unfused ? kernel_names_unfused : merged ? kernel_names_merged : kernel_names_fused;
    t->last_launches = unfused ? 5 : merged ? 1 : 2;
    if (t->W.trace) {   // debug only: reset the phase trace (mins start at ~0)
        static std::vector<unsigned long long> init;
        size_t nw = (size_t)t->grid_fused * 8 + 8;
        if (init.size() != nw) {
            init.assign(nw, 0ull);
            for (size_t c = 0; c < nw / 8; c++) init[c * 8 + 4] = ~0ull;
            init[nw - 8] = ~0ull;
        }
        cudaMemcpyAsync(t->W.trace, init.data(), nw * 8, cudaMemcpyHostToDevice, st);
    }
    mark();
    if (merged) {
        if (launch_fused(t->T, t->W, B, t->grid_fused, true, &t->bar_base, &t->epoch, st) != cudaSuccess)
            return NBA_IPSEC_ECUDA;
        mark();
        return NBA_IPSEC_OK;
    }
    if (launch_prologue(t->T, t->W, B, n_tiles, unfused, t->gridsync, st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    mark();
    if (!unfused) {
        if (launch_fused(t->T, t->W, B, t->grid_fused, false, &t->bar_base, &t->epoch, st) != cudaSuccess)
            return NBA_IPSEC_ECUDA;
        mark();
        return NBA_IPSEC_OK;
    }
    if (launch_gather(t->T, t->W, B, n_tiles, (uint32_t)t->grid_aes, st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    mark();
    if (launch_aes(t->T, t->W, B, t->grid_aes, st) != cudaSuccess) return NBA_IPSEC_ECUDA;
    mark();
    if (launch_hmac(t->T, t->W, B, st) != cudaSuccess) return NBA_IPSEC_ECUDA;
    mark();
    if (launch_scatter(t->T, t->W, B, n_stiles, st) != cudaSuccess) return NBA_IPSEC_ECUDA;
    mark();
    return NBA_IPSEC_OK;
}

int nba_ipsec_process_batch(nba_ipsec_sa_table *t, const nba_ipsec_batch *b, void *cuda_stream)
{
    if (!t || !b) return NBA_IPSEC_EINVAL;
    if (b->n_pkts > t->max_batch) return NBA_IPSEC_EINVAL;
    if (b->n_pkts == 0) return NBA_IPSEC_OK;
    if (!b->in_buf || !b->in_off || !b->in_len || !b->out_buf || !b->out_off || !b->out_len)
        return NBA_IPSEC_EINVAL;
    if (!b->sa_idx && !t->flow_table) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    const uint32_t *sa_idx = b->sa_idx;
    const bool merged = t->pipeline == NBA_IPSEC_PIPE_FUSED && t->allow_merged &&
                        fused_merged_ok(b->n_pkts, t->grid_fused);
    if (!sa_idx && !merged) {   // the SAs come from the flow table
        FlowArgs A{b->in_buf, b->in_off, b->in_len, t->flow_sa, b->n_pkts};
        if (launch_flow_lookup(t->flow_table, t->flow_mask, A, st) != cudaSuccess)
            return NBA_IPSEC_ECUDA;
        sa_idx = t->flow_sa;
    }
    // (the one-kernel path looks the SAs up itself, in its prologue)
    BatchArgs B{b->in_buf, b->in_off, b->in_len, sa_idx, b->out_buf, b->out_off, b->out_len,
                b->n_pkts, t->flow_table, t->flow_mask};
    return enqueue(t, B, st);
}

// ---- batch rings: the path for a fixed set of batch slots as one CUDA graph ----

struct nba_ipsec_ring {
    nba_ipsec_sa_table *t = nullptr;
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t exec = nullptr;
    uint32_t n_slots = 0;
    // persistent form (every slot takes the one-kernel path): the slots'
    // arguments on the device and the second count-matrix buffer
    BatchArgs *d_slots = nullptr;
    uint16_t *hist_b = nullptr;
    // persistent inbound form: slots on the device, the second replay hash
    InBatchArgs *d_in_slots = nullptr;
    unsigned long long *hkey_b = nullptr;
    uint32_t *hval_b = nullptr;
    InPipeBufs in_bufs = {};             // pipelined inbound form (hk1 / hv1 = hkey_b / hval_b)
    uint32_t in_hmask = 0;
    bool pipe = false;                   // software-pipelined form (k_fused_ring_pipe)
    bool free_run = false;               //   its free-running-lanes variant (k_fused_ring_free)
    bool in_pipe = false;                // inbound: software-pipelined form (k_in_fused_ring_pipe)
    bool pipe_ok = false;                // every slot fits the pipelined form
    bool roles = false;                  // role-split form (k_fused_ring_roles)
    bool roles_ok = false;               // every slot fits it (buffers allocated)
    RolesBufs rq = {};                   //   its hand-off counters, records, per-SA totals
    uint64_t flow_gen = 0;               // the table's flow-table generation when recorded
    uint32_t cursor = 0;                 // the slot the next run_batches starts at
    unsigned long long *ts = nullptr;    // per-batch timestamps (caller's device buffer)
    uint32_t ts_cap = 0;
    // graph form: the slots, for runs that do not start at slot 0 / end mid-rotation
    std::vector<nba_ipsec_batch> h_slots;
    std::vector<nba_ipsec_in_batch> h_in_slots;
};

int nba_ipsec_ring_create(nba_ipsec_sa_table *t, const nba_ipsec_batch *slots, uint32_t n_slots,
                          nba_ipsec_ring **out)
{
    if (!t || !slots || !out || n_slots == 0 || n_slots > 4096) return NBA_IPSEC_EINVAL;
    *out = nullptr;
    if (t->prof || t->W.trace) return NBA_IPSEC_EINVAL;   // host-side per-batch state
    for (uint32_t i = 0; i < n_slots; i++) {
        const nba_ipsec_batch &b = slots[i];
        if (b.n_pkts > t->max_batch || !b.in_buf || !b.in_off || !b.in_len || !b.out_buf ||
            !b.out_off || !b.out_len || (!b.sa_idx && !t->flow_table))
            return NBA_IPSEC_EINVAL;
    }
    DeviceGuard g(t->device);
    nba_ipsec_ring *r = new (std::nothrow) nba_ipsec_ring();
    if (!r) return NBA_IPSEC_ENOMEM;
    r->t = t;
    r->n_slots = n_slots;
    r->flow_gen = t->flow_gen;
    r->h_slots.assign(slots, slots + n_slots);
    // persistent form: one cooperative launch walks all batches of a run
    bool persist = !std::getenv("NBA_IPSEC_RING_GRAPH") && t->pipeline == NBA_IPSEC_PIPE_FUSED &&
                   t->allow_merged;
    for (uint32_t i = 0; i < n_slots && persist; i++)
        persist = slots[i].n_pkts > 0 && fused_merged_ok(slots[i].n_pkts, t->grid_fused);
    if (persist) {
        // software-pipelined form when every slot fits it (sa_idx given, <= 448
        // packets per CTA); nba_ipsec_ring_set_form switches between the two
        // persistent forms (measured, same box: 64 B 25.9 -> 23.7 us, 1514 B
        // 194.4 -> 193.3 us, IMIX 92.2 -> 97.2 us)
        r->pipe_ok = true;
        for (uint32_t i = 0; i < n_slots && r->pipe_ok; i++)
            r->pipe_ok = slots[i].sa_idx && fused_pipe_ok(slots[i].n_pkts, t->grid_fused);
        r->pipe = r->pipe_ok && !std::getenv("NBA_IPSEC_RING_NOPIPE");
        r->free_run = r->pipe && std::getenv("NBA_IPSEC_RING_FREE");
        // role-split form: sequencer CTAs + lane CTAs (every slot with SA indices,
        // <= 512 packets per lane CTA, n_sa <= ROLES_MAX_SA).  The default for
        // rings whose every slot holds packets of one length up to 1010 bytes
        // (1024-B frames) and for mixed-length rings of more than ROLES_NREC
        // slots (sorted mode): measured per 65,536-packet batch against the
        // pipelined form (tools/ring_forms.py, K = 200) 64 B 20.4 vs 22.2 us,
        // 128 B 28.9 vs 33.1, 256 B 43.2 vs 47.4, 512 B 74.2 vs 76.5, 1024 B
        // 132.9 vs 133.8, 1514 B 190.7 vs 189.0, IMIX (sorted) 69.2 vs 88.2.
        // Sequencers: 6 for packets of <= 114 bytes and mixed rings (the
        // sequencers must keep ahead of the lanes), else 4 (NBA_IPSEC_ROLES_P
        // overrides; NBA_IPSEC_RING_ROLES=0/1 forces the form).
        {
            bool one_len = true, idx = true;
            uint32_t max_len = 0;
            std::vector<uint16_t> lens;
            for (uint32_t i = 0; i < n_slots && idx; i++) {
                idx = slots[i].sa_idx != nullptr;
                lens.resize(slots[i].n_pkts);
                if (!idx || cudaMemcpy(lens.data(), slots[i].in_len, lens.size() * sizeof(uint16_t),
                                       cudaMemcpyDefault) != cudaSuccess) {
                    one_len = false;
                    break;
                }
                for (uint16_t v : lens) {
                    one_len = one_len && v == lens[0];
                    max_len = std::max<uint32_t>(max_len, v);
                }
            }
            const char *pe = std::getenv("NBA_IPSEC_ROLES_P");
            const uint32_t npro = pe ? (uint32_t)std::max(1, std::atoi(pe))
                                     : (max_len <= 114u || !one_len ? 6u : 4u);
            r->roles_ok = idx;
            for (uint32_t i = 0; i < n_slots && r->roles_ok; i++)
                r->roles_ok = fused_roles_ok(slots[i].n_pkts, t->n_sa, t->grid_fused, npro);
            if (r->roles_ok) {
                const uint32_t Lc = (uint32_t)t->grid_fused - npro;
                r->rq.npro = npro;
                if (cudaMalloc(&r->rq.ctl, ROLES_CTL_WORDS * sizeof(uint32_t)) != cudaSuccess ||
                    cudaMemset(r->rq.ctl, 0, ROLES_CTL_WORDS * sizeof(uint32_t)) != cudaSuccess ||
                    cudaMalloc(&r->rq.rec, (size_t)ROLES_NREC * Lc * 512u * sizeof(uint4)) != cudaSuccess ||
                    cudaMalloc(&r->rq.cum, (size_t)Lc * 16u * sizeof(uint32_t)) != cudaSuccess ||
                    cudaMemset(r->rq.cum, 0, (size_t)Lc * 16u * sizeof(uint32_t)) != cudaSuccess ||
                    cudaMalloc(&r->rq.ptot, (size_t)2u * npro * t->n_sa * sizeof(uint32_t)) != cudaSuccess ||
                    cudaMalloc(&r->rq.scratch, (size_t)Lc * 256u) != cudaSuccess ||
                    cudaMalloc(&r->rq.hist0, (size_t)t->n_sa * t->grid_fused * sizeof(uint32_t)) != cudaSuccess ||
                    cudaMalloc(&r->rq.tot0, (size_t)t->n_sa * sizeof(uint32_t)) != cudaSuccess ||
                    cudaMalloc(&r->rq.rows0, (size_t)t->grid_fused * 16u * t->n_sa * sizeof(uint16_t)) != cudaSuccess ||
                    cudaMalloc(&r->rq.rank0, (size_t)t->grid_fused * 512u * sizeof(uint16_t)) != cudaSuccess) {
                    nba_ipsec_ring_destroy(r);
                    return NBA_IPSEC_ENOMEM;
                }
                // sequencers stage SA indices / lengths by bulk copy when every slot's
                // arrays are 16-byte aligned
                r->rq.stage = 1u;
                for (uint32_t i = 0; i < n_slots; i++)
                    if ((reinterpret_cast<uintptr_t>(slots[i].sa_idx) | reinterpret_cast<uintptr_t>(slots[i].in_len)) & 15u)
                        r->rq.stage = 0u;
                if (std::getenv("NBA_IPSEC_ROLES_NOSTAGE")) r->rq.stage = 0u;
                // mixed lengths: per-batch length-sorted lane slots (a packet slot may
                // change lanes between uses of a ring slot: needs n_slots > ROLES_NREC)
                r->rq.sorted = (!one_len && n_slots > ROLES_NREC) ? 1u : 0u;
                const char *rs = std::getenv("NBA_IPSEC_ROLES_SORTED");
                if (rs) r->rq.sorted = (std::atoi(rs) != 0 && n_slots > ROLES_NREC) ? 1u : 0u;
                // fixed-slot mode: every CTA numbers a launch's first batch (its row
                // scans cover up to 160 CTAs)
                r->rq.boot = (!r->rq.sorted && t->grid_fused <= 160 && !std::getenv("NBA_IPSEC_ROLES_NOBOOT"))
                                 ? 1u : 0u;
                const char *re = std::getenv("NBA_IPSEC_RING_ROLES");
                r->roles = re ? std::atoi(re) != 0 : ((one_len && max_len <= 1010u) || r->rq.sorted);
            }
        }
        std::vector<BatchArgs> hb(n_slots);
        for (uint32_t i = 0; i < n_slots; i++) {
            const nba_ipsec_batch &b = slots[i];
            hb[i] = BatchArgs{b.in_buf, b.in_off, b.in_len, b.sa_idx, b.out_buf, b.out_off,
                              b.out_len, b.n_pkts, t->flow_table, t->flow_mask};
        }
        const size_t hb_bytes = (size_t)t->grid_fused * t->n_sa * sizeof(uint16_t);
        if (cudaMalloc(&r->d_slots, n_slots * sizeof(BatchArgs)) != cudaSuccess ||
            cudaMalloc(&r->hist_b, hb_bytes) != cudaSuccess ||
            cudaMemset(r->hist_b, 0, hb_bytes) != cudaSuccess ||
            cudaMemcpy(r->d_slots, hb.data(), n_slots * sizeof(BatchArgs), cudaMemcpyHostToDevice) !=
                cudaSuccess) {
            nba_ipsec_ring_destroy(r);
            return NBA_IPSEC_ENOMEM;
        }
        *out = r;
        return NBA_IPSEC_OK;
    }
    cudaStream_t cs = nullptr;
    cudaError_t e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
    int rc = NBA_IPSEC_OK;
    if (e == cudaSuccess) e = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal);
    if (e == cudaSuccess) {
        // every launch of the path reads its per-batch state (SA counters, the
        // one-kernel path's barrier base and epoch) from the device, so the
        // captured kernels are valid for any number of replays
        for (uint32_t i = 0; i < n_slots && rc == NBA_IPSEC_OK; i++)
            if (slots[i].n_pkts) rc = nba_ipsec_process_batch(t, &slots[i], cs);
        cudaGraph_t gr = nullptr;
        const cudaError_t e2 = cudaStreamEndCapture(cs, &gr);
        if (e2 != cudaSuccess && rc == NBA_IPSEC_OK) rc = NBA_IPSEC_ECUDA;
        r->graph = gr;
        if (rc == NBA_IPSEC_OK && cudaGraphInstantiate(&r->exec, r->graph, 0) != cudaSuccess)
            rc = NBA_IPSEC_ECUDA;
    } else {
        rc = NBA_IPSEC_ECUDA;
    }
    if (cs) cudaStreamDestroy(cs);
    if (rc != NBA_IPSEC_OK) {
        nba_ipsec_ring_destroy(r);
        return rc;
    }
    *out = r;
    return NBA_IPSEC_OK;
}

int nba_ipsec_ring_create_inbound(nba_ipsec_sa_table *t, const nba_ipsec_in_batch *slots,
                                  uint32_t n_slots, nba_ipsec_ring **out)
{
    if (!t || !slots || !out || n_slots == 0 || n_slots > 4096) return NBA_IPSEC_EINVAL;
    *out = nullptr;
    if (t->prof || t->W.trace || !t->in_enabled) return NBA_IPSEC_EINVAL;
    for (uint32_t i = 0; i < n_slots; i++) {
        const nba_ipsec_in_batch &b = slots[i];
        if (b.n_pkts > t->max_batch || !b.in_buf || !b.in_off || !b.in_len || !b.sa_idx ||
            !b.out_buf || !b.out_off || !b.out_len)
            return NBA_IPSEC_EINVAL;
    }
    DeviceGuard g(t->device);
    nba_ipsec_ring *r = new (std::nothrow) nba_ipsec_ring();
    if (!r) return NBA_IPSEC_ENOMEM;
    r->t = t;
    r->n_slots = n_slots;
    r->flow_gen = t->flow_gen;
    r->h_in_slots.assign(slots, slots + n_slots);
    // Forms: the software-pipelined persistent ring (k_in_fused_ring_pipe)
    // when every slot fits it (<= 448 packets per SM) and every packet is
    // small (outer length <= IN_PIPE_MAX_LEN: uniform small-packet traffic),
    // otherwise a CUDA graph of one-kernel launches.  Measured per batch,
    // graph / pipelined (profiles/ab/r02aq_inbound_sweep.txt, r02ap):
    // 64 B 39.7 / 31.8 us, 128 B 50.4 / 42.3, 256 B 63.6 / 58.2, 512 B
    // 93.7 / 92.3, 1024 B 152.8 / 156.6, 1514 B 210 / 221, IMIX 101 / 130
    // (the pipelined form has 14 lane warps, and its CTAs are coupled every
    // batch through the replay's barriers, so a mix of lengths costs it the
    // slowest CTA's lanes).  Overrides at creation: NBA_IPSEC_RING_IN_PIPE=1
    // (pipelined whenever it fits) or =0 (never), NBA_IPSEC_RING_IN_PERSIST
    // (the plain persistent ring), NBA_IPSEC_RING_GRAPH (the graph).
    const char *pipe_env = std::getenv("NBA_IPSEC_RING_IN_PIPE");
    const bool graph_only = std::getenv("NBA_IPSEC_RING_GRAPH") != nullptr || !t->allow_merged;
    bool persist = std::getenv("NBA_IPSEC_RING_IN_PERSIST") && !graph_only;
    bool pipe = !graph_only && !persist && !(pipe_env && pipe_env[0] == '0');
    uint32_t nmax = 0;
    for (uint32_t i = 0; i < n_slots; i++) {
        pipe = pipe && in_pipe_ok(slots[i].n_pkts, t->grid_fused);
        persist = persist && slots[i].n_pkts > 0 && in_merged_ok(slots[i].n_pkts, t->grid_fused);
        nmax = std::max(nmax, slots[i].n_pkts);
    }
    if (pipe && !(pipe_env && pipe_env[0] == '1')) {
        // the automatic choice: the longest outer length over the slots
        std::vector<uint16_t> len(nmax);
        for (uint32_t i = 0; i < n_slots && pipe; i++) {
            if (cudaMemcpy(len.data(), slots[i].in_len, slots[i].n_pkts * sizeof(uint16_t),
                           cudaMemcpyDeviceToHost) != cudaSuccess) {
                delete r;
                return NBA_IPSEC_ECUDA;
            }
            for (uint32_t k = 0; k < slots[i].n_pkts && pipe; k++) pipe = len[k] <= IN_PIPE_MAX_LEN;
        }
    }
    r->in_pipe = pipe;
    if (pipe || persist) {
        uint32_t hmask = 1023;   // one hash size for every slot: the largest batch's
        while (hmask + 1ull < 2ull * nmax) hmask = hmask * 2 + 1;
        r->in_hmask = hmask;
        std::vector<InBatchArgs> hb(n_slots);
        for (uint32_t i = 0; i < n_slots; i++) {
            const nba_ipsec_in_batch &b = slots[i];
            hb[i] = InBatchArgs{b.in_buf, b.in_off, b.in_len, b.sa_idx, b.out_buf, b.out_off,
                                b.out_len, b.status, b.n_pkts};
        }
        const size_t hc = t->in_hcap;
        if (cudaMalloc(&r->d_in_slots, n_slots * sizeof(InBatchArgs)) != cudaSuccess ||
            cudaMalloc(&r->hkey_b, hc * sizeof(unsigned long long)) != cudaSuccess ||
            cudaMalloc(&r->hval_b, hc * sizeof(uint32_t)) != cudaSuccess ||
            cudaMemcpy(r->d_in_slots, hb.data(), n_slots * sizeof(InBatchArgs),
                       cudaMemcpyHostToDevice) != cudaSuccess) {
            nba_ipsec_ring_destroy(r);
            return NBA_IPSEC_ENOMEM;
        }
        if (pipe) {
            InPipeBufs &P = r->in_bufs;
            P.hk1 = r->hkey_b;
            P.hv1 = r->hval_b;
            if (cudaMalloc(&P.hk2, hc * sizeof(unsigned long long)) != cudaSuccess ||
                cudaMalloc(&P.hv2, hc * sizeof(uint32_t)) != cudaSuccess ||
                cudaMalloc(&P.hk3, hc * sizeof(unsigned long long)) != cudaSuccess ||
                cudaMalloc(&P.hv3, hc * sizeof(uint32_t)) != cudaSuccess ||
                cudaMalloc(&P.scr, (size_t)t->grid_fused * 448u /* PIPE_MAX_PPC */ * sizeof(uint4)) != cudaSuccess) {
                nba_ipsec_ring_destroy(r);
                return NBA_IPSEC_ENOMEM;
            }
        }
        *out = r;
        return NBA_IPSEC_OK;
    }
    cudaStream_t cs = nullptr;
    int rc = NBA_IPSEC_OK;
    if (cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
        rc = NBA_IPSEC_ECUDA;
    } else {
        for (uint32_t i = 0; i < n_slots && rc == NBA_IPSEC_OK; i++)
            if (slots[i].n_pkts) rc = nba_ipsec_process_inbound(t, &slots[i], cs);
        cudaGraph_t gr = nullptr;
        if (cudaStreamEndCapture(cs, &gr) != cudaSuccess && rc == NBA_IPSEC_OK) rc = NBA_IPSEC_ECUDA;
        r->graph = gr;
        if (rc == NBA_IPSEC_OK && cudaGraphInstantiate(&r->exec, r->graph, 0) != cudaSuccess)
            rc = NBA_IPSEC_ECUDA;
    }
    if (cs) cudaStreamDestroy(cs);
    if (rc != NBA_IPSEC_OK) {
        nba_ipsec_ring_destroy(r);
        return rc;
    }
    *out = r;
    return NBA_IPSEC_OK;
}

// n_batches batches of the ring starting at slot `first` (persistent forms:
// one launch; graph form: whole rotations from slot 0 replay the graph, the
// other batches are launched one by one).
static int ring_launch(nba_ipsec_ring *r, uint32_t first, uint32_t n_batches, cudaStream_t st)
{
    nba_ipsec_sa_table *t = r->t;
    if (n_batches == 0) return NBA_IPSEC_OK;
    if (r->ts) {
#ifdef NBA_RING_TRACE   // debug variant: [n_batches][grid][8] phase stamps
        const size_t need = (size_t)n_batches * t->grid_fused * 16u;
#elif defined(NBA_ROLES_TRACE)
        const size_t need = (size_t)n_batches * 9u + 1u + 4u * 4u * 512u * 2u;   // + roles stamps, lanes
#else
        const size_t need = (size_t)n_batches + 1u;
#endif
        if (need > r->ts_cap) return NBA_IPSEC_EINVAL;
        if (cudaMemsetAsync(r->ts, 0, need * sizeof(unsigned long long), st) != cudaSuccess)
            return NBA_IPSEC_ECUDA;
    }
    const RingRun R{r->n_slots, first, n_batches, r->ts};
    if (r->d_in_slots)
        return (r->in_pipe ? launch_in_fused_ring_pipe(t->T, t->S, r->d_in_slots, R, r->in_hmask,
                                                       r->in_bufs, t->grid_fused, st)
                           : launch_in_fused_ring(t->T, t->S, r->d_in_slots, R, r->in_hmask,
                                                  r->hkey_b, r->hval_b, t->grid_fused, st)) ==
                       cudaSuccess
                   ? NBA_IPSEC_OK
                   : NBA_IPSEC_ECUDA;
    if (r->d_slots) {
        const cudaError_t e =
            r->roles    ? launch_fused_ring_roles(t->T, t->W, r->d_slots, R, r->rq, t->grid_fused, st)
            : r->free_run ? launch_fused_ring_free(t->T, t->W, r->d_slots, R, r->hist_b, t->grid_fused, st)
            : r->pipe   ? launch_fused_ring_pipe(t->T, t->W, r->d_slots, R, r->hist_b, t->grid_fused, st)
                        : launch_fused_ring(t->T, t->W, r->d_slots, R, r->hist_b, t->grid_fused, st);
        return e == cudaSuccess ? NBA_IPSEC_OK : NBA_IPSEC_ECUDA;
    }
    uint32_t k = first, left = n_batches;
    while (left) {
        if (k == 0 && left >= r->n_slots) {
            if (cudaGraphLaunch(r->exec, st) != cudaSuccess) return NBA_IPSEC_ECUDA;
            left -= r->n_slots;
            continue;
        }
        int rc = NBA_IPSEC_OK;
        if (!r->h_in_slots.empty()) {
            if (r->h_in_slots[k].n_pkts) rc = nba_ipsec_process_inbound(t, &r->h_in_slots[k], st);
        } else if (r->h_slots[k].n_pkts) {
            rc = nba_ipsec_process_batch(t, &r->h_slots[k], st);
        }
        if (rc != NBA_IPSEC_OK) return rc;
        k = (k + 1) % r->n_slots;
        left--;
    }
    return NBA_IPSEC_OK;
}

int nba_ipsec_ring_run(nba_ipsec_ring *r, uint32_t n_rounds, void *cuda_stream)
{
    if (!r || (!r->exec && !r->d_slots && !r->d_in_slots)) return NBA_IPSEC_EINVAL;
    if (r->t->flow_gen != r->flow_gen) return NBA_IPSEC_EINVAL;   // replaced: re-create the ring
    if ((uint64_t)n_rounds * r->n_slots > 0xffffffffull) return NBA_IPSEC_EINVAL;
    DeviceGuard g(r->t->device);
    return ring_launch(r, r->cursor, n_rounds * r->n_slots, static_cast<cudaStream_t>(cuda_stream));
}

int nba_ipsec_ring_run_batches(nba_ipsec_ring *r, uint32_t n_batches, void *cuda_stream)
{
    if (!r || (!r->exec && !r->d_slots && !r->d_in_slots)) return NBA_IPSEC_EINVAL;
    if (r->t->flow_gen != r->flow_gen) return NBA_IPSEC_EINVAL;
    DeviceGuard g(r->t->device);
    const int rc = ring_launch(r, r->cursor, n_batches, static_cast<cudaStream_t>(cuda_stream));
    if (rc == NBA_IPSEC_OK) r->cursor = (uint32_t)(((uint64_t)r->cursor + n_batches) % r->n_slots);
    return rc;
}

int nba_ipsec_ring_cursor(const nba_ipsec_ring *r)
{
    if (!r) return NBA_IPSEC_EINVAL;
    return (int)r->cursor;
}

int nba_ipsec_ring_set_timestamps(nba_ipsec_ring *r, unsigned long long *dev_ts, uint32_t cap)
{
    if (!r || (dev_ts && cap < 2)) return NBA_IPSEC_EINVAL;
    if (dev_ts && !r->d_slots && !r->d_in_slots) return NBA_IPSEC_EINVAL;   // persistent forms only
    r->ts = dev_ts;
    r->ts_cap = dev_ts ? cap : 0;
    return NBA_IPSEC_OK;
}

int nba_ipsec_ring_set_form(nba_ipsec_ring *r, int form)
{
    if (!r || !r->d_slots) return NBA_IPSEC_EINVAL;   // graph rings have one form
    if (form == NBA_IPSEC_RING_PERSISTENT) {
        r->pipe = r->free_run = r->roles = false;
        return NBA_IPSEC_OK;
    }
    if (form == NBA_IPSEC_RING_ROLES && r->roles_ok) {
        r->pipe = r->free_run = false;
        r->roles = true;
        return NBA_IPSEC_OK;
    }
    if ((form == NBA_IPSEC_RING_PIPELINED || form == NBA_IPSEC_RING_FREE) && r->pipe_ok) {
        r->roles = false;
        r->pipe = true;
        r->free_run = form == NBA_IPSEC_RING_FREE;
        return NBA_IPSEC_OK;
    }
    return NBA_IPSEC_EINVAL;
}

int nba_ipsec_ring_form(const nba_ipsec_ring *r)
{
    if (!r) return NBA_IPSEC_EINVAL;
    if (r->d_in_slots) return r->in_pipe ? NBA_IPSEC_RING_PIPELINED : NBA_IPSEC_RING_PERSISTENT;
    return !r->d_slots ? NBA_IPSEC_RING_GRAPH
           : r->roles    ? NBA_IPSEC_RING_ROLES
           : r->free_run ? NBA_IPSEC_RING_FREE
           : r->pipe    ? NBA_IPSEC_RING_PIPELINED
                        : NBA_IPSEC_RING_PERSISTENT;
}

int nba_ipsec_ring_destroy(nba_ipsec_ring *r)
{
    if (!r) return NBA_IPSEC_OK;
    {
        DeviceGuard g(r->t->device);
        if (r->exec) cudaGraphExecDestroy(r->exec);
        if (r->graph) cudaGraphDestroy(r->graph);
        if (r->d_slots || r->hist_b || r->d_in_slots || r->hkey_b || r->hval_b || r->rq.ctl)
            cudaDeviceSynchronize();   // a run may still be in flight
        for (void *q : {(void *)r->rq.ctl, (void *)r->rq.rec, (void *)r->rq.ptot, (void *)r->rq.scratch,
                        (void *)r->rq.cum, (void *)r->rq.hist0, (void *)r->rq.tot0, (void *)r->rq.rows0,
                        (void *)r->rq.rank0})
            if (q) cudaFree(q);
        if (r->d_slots) cudaFree(r->d_slots);
        if (r->hist_b) cudaFree(r->hist_b);
        if (r->d_in_slots) cudaFree(r->d_in_slots);
        if (r->hkey_b) cudaFree(r->hkey_b);
        if (r->hval_b) cudaFree(r->hval_b);
        for (void *q : {(void *)r->in_bufs.hk2, (void *)r->in_bufs.hv2, (void *)r->in_bufs.hk3,
                        (void *)r->in_bufs.hv3, (void *)r->in_bufs.scr})
            if (q) cudaFree(q);
    }
    delete r;
    return NBA_IPSEC_OK;
}

static void io_free(nba_ipsec_sa_table *t)
{
    for (auto &sl : t->io) {
        if (sl.in) cudaFree(sl.in);
        if (sl.out) cudaFree(sl.out);
        if (sl.meta) cudaFree(sl.meta);
        sl.in = sl.out = nullptr;
        sl.meta = nullptr;
    }
    t->io_in_bytes = t->io_out_bytes = 0;
}

int nba_ipsec_reserve_host_io(nba_ipsec_sa_table *t, uint64_t in_buf_bytes, uint64_t out_buf_bytes)
{
    if (!t) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    cudaError_t e = cudaSuccess;
    auto chk = [&](cudaError_t x) {
        if (e == cudaSuccess && x != cudaSuccess) e = x;
    };
    if (!t->s_h2d) {
        chk(cudaStreamCreateWithFlags(&t->s_h2d, cudaStreamNonBlocking));
        chk(cudaStreamCreateWithFlags(&t->s_comp, cudaStreamNonBlocking));
        chk(cudaStreamCreateWithFlags(&t->s_d2h, cudaStreamNonBlocking));
        chk(cudaEventCreateWithFlags(&t->ev_call, cudaEventDisableTiming));
        for (auto &sl : t->io) {
            chk(cudaEventCreateWithFlags(&sl.in_ready, cudaEventDisableTiming));
            chk(cudaEventCreateWithFlags(&sl.done, cudaEventDisableTiming));
            chk(cudaEventCreateWithFlags(&sl.out_done, cudaEventDisableTiming));
        }
        if (e != cudaSuccess) {
            cudaGetLastError();
            return NBA_IPSEC_ECUDA;
        }
    }
    if (in_buf_bytes <= t->io_in_bytes && out_buf_bytes <= t->io_out_bytes && t->io_ready)
        return NBA_IPSEC_OK;
    // grow: wait for batches in flight, then reallocate every slot
    cudaStreamSynchronize(t->s_h2d);
    cudaStreamSynchronize(t->s_comp);
    cudaStreamSynchronize(t->s_d2h);
    const uint64_t inb = std::max(in_buf_bytes, t->io_in_bytes);
    const uint64_t outb = std::max(out_buf_bytes, t->io_out_bytes);
    io_free(t);
    t->io_ready = false;
    // (zeroed once: the lanes' 32-byte loads may cover up to 31 bytes past
    // the copied input, and the copy-out takes the whole output range,
    // including bytes between the slots the kernels never write)
    for (auto &sl : t->io) {
        chk(cudaMalloc(&sl.in, inb + 64));
        chk(cudaMalloc(&sl.out, outb + 64));
        chk(cudaMalloc(&sl.meta, (size_t)t->max_batch * 16 + 64));
        if (e == cudaSuccess) {
            chk(cudaMemset(sl.in, 0, inb + 64));
            chk(cudaMemset(sl.out, 0, outb + 64));
        }
    }
    if (e == cudaSuccess) chk(cudaDeviceSynchronize());   // before the non-blocking streams' copies
    if (e != cudaSuccess) {
        cudaGetLastError();
        io_free(t);
        return NBA_IPSEC_ENOMEM;
    }
    t->io_in_bytes = inb;
    t->io_out_bytes = outb;
    t->io_ready = true;
    return NBA_IPSEC_OK;
}

int nba_ipsec_process_batch_host(nba_ipsec_sa_table *t, const nba_ipsec_batch *b,
                                 uint64_t in_buf_bytes, uint64_t out_buf_bytes, void *cuda_stream)
{
    if (!t || !b) return NBA_IPSEC_EINVAL;
    if (b->n_pkts > t->max_batch) return NBA_IPSEC_EINVAL;
    if (b->n_pkts == 0) return NBA_IPSEC_OK;
    if (!b->in_buf || !b->in_off || !b->in_len || !b->sa_idx || !b->out_buf || !b->out_off ||
        !b->out_len)
        return NBA_IPSEC_EINVAL;
    if (!t->io_ready || in_buf_bytes > t->io_in_bytes || out_buf_bytes > t->io_out_bytes)
        return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    auto &sl = t->io[t->io_next % nba_ipsec_sa_table::IO_DEPTH];
    t->io_next++;
    const uint32_t n = b->n_pkts;
    uint32_t *d_in_off = sl.meta;
    uint32_t *d_sa = d_in_off + t->max_batch;
    uint32_t *d_out_off = d_sa + t->max_batch;
    uint16_t *d_in_len = reinterpret_cast<uint16_t *>(d_out_off + t->max_batch);
    uint16_t *d_out_len = d_in_len + t->max_batch;
    // Per-packet metadata in page-locked host memory the device can address
    // (cudaHostAlloc'd or registered) does not go through the copy engines:
    // the four small copies in and one out cost ~50 us per 65,536-packet step
    // in copy-engine time (tools/pcie_probe.py).  The main kernels read the
    // host arrays in place over PCIe and write out_len there.  Measured per
    // 64 B step (profiles/ab/r02az_pcie.txt): in place 180.7 us, copies
    // (NBA_IPSEC_HOST_META=stage) 199.3; a pull kernel copying the four
    // arrays into the staging slot first: 192.7 on the compute stream, 317 on
    // the copy-in stream (it waits for the cooperative kernel's SMs).
    // Pageable metadata is staged with copies like in_buf.
    auto mapped = [](const void *p) -> void * {
        cudaPointerAttributes a;
        if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        return a.type == cudaMemoryTypeHost ? a.devicePointer : nullptr;
    };
    const char *hm = std::getenv("NBA_IPSEC_HOST_META");
    bool zc = !(hm && !std::strcmp(hm, "stage"));
    void *z_in_off = nullptr, *z_sa = nullptr, *z_out_off = nullptr, *z_in_len = nullptr, *z_out_len = nullptr;
    if (zc) {
        z_in_off = mapped(b->in_off);
        z_sa = mapped(b->sa_idx);
        z_out_off = mapped(b->out_off);
        z_in_len = mapped(b->in_len);
        z_out_len = mapped(b->out_len);
        zc = z_in_off && z_sa && z_out_off && z_in_len && z_out_len;
    }
    if (zc) {
        d_in_off = static_cast<uint32_t *>(z_in_off);
        d_sa = static_cast<uint32_t *>(z_sa);
        d_out_off = static_cast<uint32_t *>(z_out_off);
        d_in_len = static_cast<uint16_t *>(z_in_len);
        d_out_len = static_cast<uint16_t *>(z_out_len);
    }
    cudaError_t e = cudaSuccess;
    auto chk = [&](cudaError_t x) {
        if (e == cudaSuccess && x != cudaSuccess) e = x;
    };
    // copy-in: after this slot's previous copy-out has drained its buffers
    chk(cudaStreamWaitEvent(t->s_h2d, sl.out_done, 0));
    chk(cudaMemcpyAsync(sl.in, b->in_buf, in_buf_bytes, cudaMemcpyHostToDevice, t->s_h2d));
    if (!zc) {
        chk(cudaMemcpyAsync(d_in_off, b->in_off, n * 4ull, cudaMemcpyHostToDevice, t->s_h2d));
        chk(cudaMemcpyAsync(d_sa, b->sa_idx, n * 4ull, cudaMemcpyHostToDevice, t->s_h2d));
        chk(cudaMemcpyAsync(d_out_off, b->out_off, n * 4ull, cudaMemcpyHostToDevice, t->s_h2d));
        chk(cudaMemcpyAsync(d_in_len, b->in_len, n * 2ull, cudaMemcpyHostToDevice, t->s_h2d));
    }
    chk(cudaEventRecord(sl.in_ready, t->s_h2d));
    // compute: after the inputs and after everything the caller's stream holds
    // (keeps the SA counters in call order with device-path batches)
    chk(cudaEventRecord(t->ev_call, st));
    chk(cudaStreamWaitEvent(t->s_comp, t->ev_call, 0));
    chk(cudaStreamWaitEvent(t->s_comp, sl.in_ready, 0));
    if (e != cudaSuccess) return NBA_IPSEC_ECUDA;
    BatchArgs B{sl.in, d_in_off, d_in_len, d_sa, sl.out, d_out_off, d_out_len, n};
    int rc = enqueue(t, B, t->s_comp);
    if (rc != NBA_IPSEC_OK) return rc;
    chk(cudaEventRecord(sl.done, t->s_comp));
    chk(cudaStreamWaitEvent(st, sl.done, 0));        // later work on the caller's stream
    // copy-out
    chk(cudaStreamWaitEvent(t->s_d2h, sl.done, 0));
    chk(cudaMemcpyAsync(b->out_buf, sl.out, out_buf_bytes, cudaMemcpyDeviceToHost, t->s_d2h));
    if (!zc) chk(cudaMemcpyAsync(b->out_len, d_out_len, n * 2ull, cudaMemcpyDeviceToHost, t->s_d2h));
    chk(cudaEventRecord(sl.out_done, t->s_d2h));
    return e == cudaSuccess ? NBA_IPSEC_OK : NBA_IPSEC_ECUDA;
}

int nba_ipsec_host_wait(nba_ipsec_sa_table *t, void *cuda_stream)
{
    if (!t) return NBA_IPSEC_EINVAL;
    if (!t->s_d2h) return NBA_IPSEC_OK;
    DeviceGuard g(t->device);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    cudaError_t e = cudaEventRecord(t->ev_call, t->s_d2h);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(st, t->ev_call, 0);
    return e == cudaSuccess ? NBA_IPSEC_OK : NBA_IPSEC_ECUDA;
}

int nba_ipsec_destroy(nba_ipsec_sa_table *t)
{
    if (!t) return NBA_IPSEC_OK;
    {
        DeviceGuard g(t->device);
        cudaDeviceSynchronize();
        free_all(t);
        io_free(t);
        if (t->flow_table) cudaFree(t->flow_table);
        if (t->flow_sa) cudaFree(t->flow_sa);
        for (auto &sl : t->io) {
            if (sl.in_ready) cudaEventDestroy(sl.in_ready);
            if (sl.done) cudaEventDestroy(sl.done);
            if (sl.out_done) cudaEventDestroy(sl.out_done);
        }
        if (t->ev_call) cudaEventDestroy(t->ev_call);
        if (t->s_h2d) cudaStreamDestroy(t->s_h2d);
        if (t->s_comp) cudaStreamDestroy(t->s_comp);
        if (t->s_d2h) cudaStreamDestroy(t->s_d2h);
    }
    delete t;
    return NBA_IPSEC_OK;
}

int nba_ipsec_read_counters(nba_ipsec_sa_table *t, nba_ipsec_counters *out, void *cuda_stream)
{
    if (!t || !out) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    unsigned long long h[5];
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    if (cudaMemcpyAsync(h, t->W.counters, sizeof(h), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaStreamSynchronize(st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    out->pkts_ok = h[0];
    out->pkts_dropped = h[1];
    out->bytes_in = h[2];
    out->bytes_out = h[3];
    out->batches = h[4];
    return NBA_IPSEC_OK;
}

int nba_ipsec_read_sa_seq(nba_ipsec_sa_table *t, uint32_t *host_seq, void *cuda_stream)
{
    if (!t || !host_seq) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    if (cudaMemcpyAsync(host_seq, t->T.seq, t->n_sa * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                        st) != cudaSuccess ||
        cudaStreamSynchronize(st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    return NBA_IPSEC_OK;
}

int nba_ipsec_write_sa_seq(nba_ipsec_sa_table *t, const uint32_t *host_seq, void *cuda_stream)
{
    // counter hand-over between devices (reading L7)
    if (!t || !host_seq) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    if (cudaMemcpyAsync(t->T.seq, host_seq, t->n_sa * sizeof(uint32_t), cudaMemcpyHostToDevice,
                        st) != cudaSuccess ||
        cudaStreamSynchronize(st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    return NBA_IPSEC_OK;
}

int nba_ipsec_debug_trace(nba_ipsec_sa_table *t, uint64_t *host, uint32_t n_words)
{
    if (!t || !host) return NBA_IPSEC_EINVAL;
    if (!t->W.trace) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    size_t n = std::min<size_t>(n_words, (size_t)t->grid_fused * 8 + 64);
    if (cudaDeviceSynchronize() != cudaSuccess ||
        cudaMemcpy(host, t->W.trace, n * 8, cudaMemcpyDeviceToHost) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    return NBA_IPSEC_OK;
}

int nba_ipsec_set_pipeline(nba_ipsec_sa_table *t, int pipeline)
{
    if (!t) return NBA_IPSEC_EINVAL;
    if (pipeline != NBA_IPSEC_PIPE_UNFUSED && pipeline != NBA_IPSEC_PIPE_FUSED)
        return NBA_IPSEC_EINVAL;
    t->pipeline = pipeline;
    return NBA_IPSEC_OK;
}

int nba_ipsec_launches_per_batch(nba_ipsec_sa_table *t)
{
    if (!t) return NBA_IPSEC_EINVAL;
    return t->last_launches;
}

int nba_ipsec_inbound_launches_per_batch(nba_ipsec_sa_table *t)
{
    if (!t) return NBA_IPSEC_EINVAL;
    return (int)t->in_last_launches;
}

int nba_ipsec_profile_enable(nba_ipsec_sa_table *t, int enable)
{
    if (!t) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    for (auto &s : t->ring) s.n_ev = 0;
    t->prof = enable != 0;
    t->prof_batches = 0;
    t->prof_nk = 0;
    for (double &x : t->prof_ms) x = 0.0;
    for (double &x : t->prof_in_ms) x = 0.0;
    t->prof_in_batches = 0;
    return NBA_IPSEC_OK;
}

int nba_ipsec_profile_read(nba_ipsec_sa_table *t, double *ms, const char **names, int max,
                           int *n_kernels, uint32_t *n_batches)
{
    if (!t) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    for (int k = 0; k < PROF_RING; k++) prof_drain_set(t, t->ring[(t->ring_next + k) % PROF_RING]);
    const char **nm = t->prof_names ? t->prof_names : kernel_names_fused;
    int nk = t->prof_nk;
    for (int k = 0; k < nk && k < max; k++) {
        if (ms) ms[k] = t->prof_ms[k];
        if (names) names[k] = nm[k];
    }
    if (n_kernels) *n_kernels = nk;
    if (n_batches) *n_batches = t->prof_batches;
    return NBA_IPSEC_OK;
}

// ---- ESP inbound -----------------------------------------

// ---- flow -> SA lookup ----------------------------------

int nba_ipsec_set_flow_table(nba_ipsec_sa_table *t, const nba_ipsec_flow *flows, uint32_t n_flows)
{
    if (!t || (!flows && n_flows) || n_flows > (1u << 26)) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    t->flow_gen++;
    if (n_flows == 0) {
        cudaDeviceSynchronize();
        if (t->flow_table) cudaFree(t->flow_table);
        t->flow_table = nullptr;
        t->flow_mask = 0;
        return NBA_IPSEC_OK;
    }
    uint32_t cap = 64;
    while (cap < 2ull * n_flows) cap <<= 1;
    std::vector<uint4> tab(cap, make_uint4(0, 0, 0, 0));
    for (uint32_t k = 0; k < n_flows; k++) {
        const nba_ipsec_flow &f = flows[k];
        if (f.sa >= t->n_sa) return NBA_IPSEC_EINVAL;
        const uint32_t ports = ((uint32_t)f.sport << 16) | f.dport;
        uint32_t h = flow_hash(f.src, f.dst, ports, f.proto) & (cap - 1u);
        while (tab[h].w & FLOW_VALID) {
            if (tab[h].x == f.src && tab[h].y == f.dst && tab[h].z == ports &&
                (tab[h].w & 0xffu) == f.proto)
                return NBA_IPSEC_EINVAL;   // duplicate key
            h = (h + 1u) & (cap - 1u);
        }
        tab[h] = make_uint4(f.src, f.dst, ports, (uint32_t)f.proto | FLOW_VALID | (f.sa << 16));
    }
    cudaError_t e = cudaSuccess;
    if (!t->flow_sa) {
        e = cudaMalloc(&t->flow_sa, (size_t)t->max_batch * 4 + 64);
        if (e != cudaSuccess) {
            cudaGetLastError();
            t->flow_sa = nullptr;
            return NBA_IPSEC_ENOMEM;
        }
    }
    cudaDeviceSynchronize();   // the old table may be in use by enqueued work
    if (t->flow_table) cudaFree(t->flow_table);
    t->flow_table = nullptr;
    if (cudaMalloc(&t->flow_table, cap * sizeof(uint4)) != cudaSuccess) {
        cudaGetLastError();
        return NBA_IPSEC_ENOMEM;
    }
    if (cudaMemcpy(t->flow_table, tab.data(), cap * sizeof(uint4), cudaMemcpyHostToDevice) !=
        cudaSuccess)
        return NBA_IPSEC_ECUDA;
    t->flow_mask = cap - 1u;
    return NBA_IPSEC_OK;
}

int nba_ipsec_lookup_sa(nba_ipsec_sa_table *t, const uint8_t *in_buf, const uint32_t *in_off,
                        const uint16_t *in_len, uint32_t n_pkts, uint32_t *sa_idx,
                        void *cuda_stream)
{
    if (!t || !t->flow_table || n_pkts > t->max_batch) return NBA_IPSEC_EINVAL;
    if (n_pkts == 0) return NBA_IPSEC_OK;
    if (!in_buf || !in_off || !in_len || !sa_idx) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    FlowArgs A{in_buf, in_off, in_len, sa_idx, n_pkts};
    return launch_flow_lookup(t->flow_table, t->flow_mask, A, static_cast<cudaStream_t>(cuda_stream)) ==
                   cudaSuccess
               ? NBA_IPSEC_OK
               : NBA_IPSEC_ECUDA;
}

// ---- single-ingress redistribution ----------------------

int nba_ipsec_route_workspace_bytes(uint32_t max_pkts, uint32_t world, uint64_t *bytes)
{
    if (!bytes || world == 0 || world > 8 || max_pkts > NBA_IPSEC_MAX_BATCH) return NBA_IPSEC_EINVAL;
    *bytes = route_workspace_bytes(max_pkts, world);
    return NBA_IPSEC_OK;
}

int nba_ipsec_route_pack_map(const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                             const uint32_t *sa_global, uint32_t n_pkts, uint32_t n_sa_total,
                             const uint32_t *sa_map, uint32_t world, void *workspace,
                             uint8_t *send_buf, uint16_t *send_len, uint32_t *send_sa,
                             uint64_t *dest_counts, uint64_t *dest_bytes, void *cuda_stream)
{
    if (world == 0 || world > 8 || n_pkts > NBA_IPSEC_MAX_BATCH) return NBA_IPSEC_EINVAL;
    if (!dest_counts || !dest_bytes) return NBA_IPSEC_EINVAL;
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    if (n_pkts == 0) {
        return cudaMemsetAsync(dest_counts, 0, (world + 1) * 8ull, st) == cudaSuccess &&
                       cudaMemsetAsync(dest_bytes, 0, (world + 1) * 8ull, st) == cudaSuccess
                   ? NBA_IPSEC_OK
                   : NBA_IPSEC_ECUDA;
    }
    if (!in_buf || !in_off || !in_len || !sa_global || !workspace || !send_buf || !send_len ||
        !send_sa)
        return NBA_IPSEC_EINVAL;
    return launch_route(in_buf, in_off, in_len, sa_global, n_pkts, n_sa_total, sa_map, world,
                        workspace, send_buf, send_len, send_sa,
                        reinterpret_cast<unsigned long long *>(dest_counts),
                        reinterpret_cast<unsigned long long *>(dest_bytes), st) == cudaSuccess
               ? NBA_IPSEC_OK
               : NBA_IPSEC_ECUDA;
}

int nba_ipsec_route_dispatch(const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                             const uint32_t *sa_global, uint32_t n_pkts, uint32_t n_sa_total,
                             const uint32_t *sa_map, uint32_t world, void *workspace,
                             const nba_ipsec_peer_rx *rx, uint64_t cap_pkts, uint64_t cap_bytes,
                             uint64_t *dest_counts, uint64_t *dest_bytes, void *cuda_stream)
{
    if (world == 0 || world > 8 || n_pkts > NBA_IPSEC_MAX_BATCH) return NBA_IPSEC_EINVAL;
    if (!dest_counts || !dest_bytes || !rx) return NBA_IPSEC_EINVAL;   // any capacity: prefix kept
    if (n_pkts && (!in_buf || !in_off || !in_len || !sa_global || !workspace))
        return NBA_IPSEC_EINVAL;
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    // (an empty batch runs only the scan, which writes every receiver's zero counts)
    if (!workspace) return NBA_IPSEC_EINVAL;
    return launch_route(in_buf, in_off, in_len, sa_global, n_pkts, n_sa_total, sa_map, world,
                        workspace, nullptr, nullptr, nullptr,
                        reinterpret_cast<unsigned long long *>(dest_counts),
                        reinterpret_cast<unsigned long long *>(dest_bytes), st, rx, cap_pkts,
                        cap_bytes) == cudaSuccess
               ? NBA_IPSEC_OK
               : NBA_IPSEC_ECUDA;
}

int nba_ipsec_route_pack(const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                         const uint32_t *sa_global, uint32_t n_pkts, uint32_t n_sa_total,
                         uint32_t world, void *workspace, uint8_t *send_buf, uint16_t *send_len,
                         uint32_t *send_sa, uint64_t *dest_counts, uint64_t *dest_bytes,
                         void *cuda_stream)
{
    return nba_ipsec_route_pack_map(in_buf, in_off, in_len, sa_global, n_pkts, n_sa_total, nullptr,
                                    world, workspace, send_buf, send_len, send_sa, dest_counts,
                                    dest_bytes, cuda_stream);
}

int nba_ipsec_enable_inbound(nba_ipsec_sa_table *t)
{
    if (!t) return NBA_IPSEC_EINVAL;
    if (t->in_enabled) return NBA_IPSEC_OK;
    DeviceGuard g(t->device);
    const uint32_t n_sa = t->n_sa, M = t->max_batch;
    uint32_t hcap = 1024;
    while (hcap < 2ull * M) hcap <<= 1;
    InState &S = t->S;
    cudaError_t e = cudaSuccess;
    auto chk = [&](cudaError_t x) {
        if (e == cudaSuccess && x != cudaSuccess) e = x;
    };
    chk(dalloc(t, &S.top, n_sa));
    chk(dalloc(t, &S.top_prev, n_sa));
    chk(dalloc(t, &S.bmp, n_sa));
    chk(dalloc(t, &S.bmp_prev, n_sa));
    chk(dalloc(t, &S.flags, M));
    chk(dalloc(t, &S.seq, M));
    chk(dalloc(t, &S.lmax, M));
    // columns: the three-kernel path's tiles, or the one-kernel path's CTAs
    const size_t cols = std::max<size_t>(t->max_tiles, (size_t)t->grid_fused);
    chk(dalloc(t, &S.hmax, cols * n_sa));
    chk(dalloc(t, &S.pmx, cols * n_sa));
    chk(dalloc(t, &S.hkey, hcap));
    chk(dalloc(t, &S.hval, hcap));
    for (int k = 0; k < 2; k++) {
        chk(dalloc(t, &t->HP.hk[k], hcap));
        chk(dalloc(t, &t->HP.hv[k], hcap));
    }
    chk(dalloc(t, &S.counters, N_IN_COUNTERS));
    chk(dalloc(t, &S.ctl, 8));
    chk(dalloc(t, &t->in_top0, n_sa));
    chk(dalloc(t, &t->in_bmp0, n_sa));
    if (e == cudaSuccess) {
        for (int k = 0; k < 2; k++) {          // the one-kernel path's hashes start empty
            chk(cudaMemset(t->HP.hk[k], 0xff, hcap * sizeof(unsigned long long)));
            chk(cudaMemset(t->HP.hv[k], 0xff, hcap * sizeof(uint32_t)));
        }
        // reading B6: the window starts at the SA's seq, everything <= seq seen
        std::vector<unsigned long long> bmp(n_sa);
        for (uint32_t s = 0; s < n_sa; s++) bmp[s] = t->seq0[s] ? ~0ull : 0ull;
        chk(cudaMemcpy(S.top, t->seq0.data(), n_sa * 4ull, cudaMemcpyHostToDevice));
        chk(cudaMemcpy(S.bmp, bmp.data(), n_sa * 8ull, cudaMemcpyHostToDevice));
        chk(cudaMemcpy(t->in_top0, t->seq0.data(), n_sa * 4ull, cudaMemcpyHostToDevice));
        chk(cudaMemcpy(t->in_bmp0, bmp.data(), n_sa * 8ull, cudaMemcpyHostToDevice));
    }
    if (e == cudaSuccess) chk(setup_inbound_attributes(n_sa, t->max_tiles, t->num_sms, &t->in_gridsync));
    if (std::getenv("NBA_IPSEC_NO_GRIDSYNC")) t->in_gridsync = false;
    if (e == cudaSuccess) chk(cudaDeviceSynchronize());
    if (e != cudaSuccess) {
        cudaGetLastError();
        return e == cudaErrorMemoryAllocation ? NBA_IPSEC_ENOMEM : NBA_IPSEC_ECUDA;
    }
    t->in_hcap = hcap;
    t->in_enabled = true;
    return NBA_IPSEC_OK;
}

int nba_ipsec_process_inbound(nba_ipsec_sa_table *t, const nba_ipsec_in_batch *b, void *cuda_stream)
{
    if (!t || !b) return NBA_IPSEC_EINVAL;
    if (!t->in_enabled || b->n_pkts > t->max_batch) return NBA_IPSEC_EINVAL;
    if (b->n_pkts == 0) return NBA_IPSEC_OK;
    if (!b->in_buf || !b->in_off || !b->in_len || !b->sa_idx || !b->out_buf || !b->out_off ||
        !b->out_len)
        return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    const uint32_t n = b->n_pkts;
    uint32_t hmask = 1023;
    while (hmask + 1ull < 2ull * n) hmask = hmask * 2 + 1;
    const uint32_t n_tiles = (n + PTILE - 1) / PTILE;
    InBatchArgs B{b->in_buf, b->in_off, b->in_len, b->sa_idx, b->out_buf, b->out_off, b->out_len,
                  b->status, n};
    ProfSet *ps = nullptr;
    if (t->prof) {
        ps = &t->ring[t->ring_next];
        prof_drain_set(t, *ps);
        t->ring_next = (t->ring_next + 1) % PROF_RING;
        for (int k = 0; k < MAX_KERNELS + 1; k++)
            if (!ps->ev[k]) cudaEventCreate(&ps->ev[k]);
        ps->n_ev = 0;
        ps->inbound = true;
    }
    auto mark = [&]() {
        if (ps) cudaEventRecord(ps->ev[ps->n_ev++], st);
    };
    mark();
    // one kernel when the batch fits one super-round per CTA (the replay
    // decision inside, behind two grid barriers); else three kernels
    const bool merged = t->allow_merged && in_merged_ok(n, t->grid_fused);
    t->in_last_launches = merged ? 1 : 3;
    if (launch_in_fused(t->T, t->S, t->HP, B, t->grid_fused, hmask, t->in_hcap - 1u, merged,
                        &t->in_bar_base, st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    mark();
    if (merged) return NBA_IPSEC_OK;
    if (launch_in_replay(t->T, t->S, B, n_tiles, hmask, t->in_gridsync, st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    mark();
    if (launch_in_decide(t->T, t->S, B, n_tiles, hmask, st) != cudaSuccess) return NBA_IPSEC_ECUDA;
    mark();
    return NBA_IPSEC_OK;
}

int nba_ipsec_reset_inbound(nba_ipsec_sa_table *t, void *cuda_stream)
{
    if (!t || !t->in_enabled) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    if (cudaMemcpyAsync(t->S.top, t->in_top0, t->n_sa * 4ull, cudaMemcpyDeviceToDevice, st) !=
            cudaSuccess ||
        cudaMemcpyAsync(t->S.bmp, t->in_bmp0, t->n_sa * 8ull, cudaMemcpyDeviceToDevice, st) !=
            cudaSuccess)
        return NBA_IPSEC_ECUDA;
    return NBA_IPSEC_OK;
}

int nba_ipsec_read_in_counters(nba_ipsec_sa_table *t, nba_ipsec_in_counters *out, void *cuda_stream)
{
    if (!t || !out || !t->in_enabled) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    unsigned long long h[N_IN_COUNTERS];
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    if (cudaMemcpyAsync(h, t->S.counters, sizeof(h), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaStreamSynchronize(st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    out->pkts_ok = h[0];
    out->drop_sa = h[1];
    out->drop_format = h[2];
    out->drop_replay = h[3];
    out->drop_auth = h[4];
    out->drop_trailer = h[5];
    out->bytes_in = h[6];
    out->bytes_out = h[7];
    out->batches = h[8];
    return NBA_IPSEC_OK;
}

int nba_ipsec_read_replay_window(nba_ipsec_sa_table *t, uint32_t *top, uint64_t *bitmap,
                                 void *cuda_stream)
{
    if (!t || !top || !bitmap || !t->in_enabled) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    if (cudaMemcpyAsync(top, t->S.top, t->n_sa * 4ull, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaMemcpyAsync(bitmap, t->S.bmp, t->n_sa * 8ull, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaStreamSynchronize(st) != cudaSuccess)
        return NBA_IPSEC_ECUDA;
    return NBA_IPSEC_OK;
}

int nba_ipsec_profile_read_inbound(nba_ipsec_sa_table *t, double *ms, const char **names, int max,
                                   int *n_kernels, uint32_t *n_batches)
{
    static const char *nm[3] = {"in_fused", "in_replay", "in_decide"};
    if (!t) return NBA_IPSEC_EINVAL;
    DeviceGuard g(t->device);
    for (int k = 0; k < PROF_RING; k++) prof_drain_set(t, t->ring[(t->ring_next + k) % PROF_RING]);
    for (int k = 0; k < 3 && k < max; k++) {
        if (ms) ms[k] = t->prof_in_ms[k];
        if (names) names[k] = nm[k];
    }
    if (n_kernels) *n_kernels = (int)t->in_last_launches;
    if (n_batches) *n_batches = t->prof_in_batches;
    return NBA_IPSEC_OK;
}

}  // extern "C"
