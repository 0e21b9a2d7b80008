// alb.cpp -- adaptive load balancer of the SA split across devices
// (§3.4 "Adaptive CPU/GPU Load Balancing").
//
// NBA hill-climbs the offloading fraction w in steps of delta on the measured
// throughput (moving average), waits for the workers to apply each change and
// keeps perturbing w by delta so it follows workload changes.  On a B200 box
// the split being balanced is the ownership of SAs between GPUs (with single
// ingress, a GPU processes exactly the packets of the SAs it owns, S§8(e)):
// w is the fraction of a node's SAs that go to its right half of devices, a
// binary tree of controllers covers up to 8 devices.  Readings L1-L7 of
// DESIGN.md §2 fix what the paper leaves open; the controller is host code
// (no device work), exported through include/nba_ipsec.h.
//
// Decisions are exact: samples are integers (packets, nanoseconds) and the
// throughput comparison is a 128-bit cross-multiplication, so the trajectory
// of w is a deterministic function of the samples.
#include <cstdint>
#include <cstdlib>
#include <new>
#include <vector>

#include "nba_ipsec.h"

struct nba_ipsec_alb {
    nba_ipsec_alb_params p;
    uint32_t k;          // current step: w = k / p.steps
    int dir;             // +1 / -1
    bool started;
    bool waiting;        // true: in the waiting interval after an update (L3)
    uint64_t t_end;      // end of the wait / of the observation
    // moving-average window (L2): ring of the last `history` samples
    std::vector<uint64_t> rp, rt;
    uint32_t head, count;
    unsigned __int128 sum_p, sum_t;
    bool have_prev;
    uint64_t prev_p, prev_t;
    uint64_t updates;
};

namespace {

uint64_t wait_ns(const nba_ipsec_alb &a, uint32_t k)
{
    // L4: waiting interval grows linearly from wait_min (w = 0) to wait_max
    // (w = 100%) update intervals
    const uint64_t span = a.p.wait_max - a.p.wait_min;
    const uint64_t n = a.p.wait_min + span * k / a.p.steps;
    return n * a.p.update_ns;
}

void ring_clear(nba_ipsec_alb &a)
{
    a.head = a.count = 0;
    a.sum_p = a.sum_t = 0;
}

void ring_push(nba_ipsec_alb &a, uint64_t p, uint64_t t)
{
    const uint32_t H = a.p.history;
    if (a.count == H) {              // evict the oldest sample
        const uint32_t old = (a.head + H - a.count) % H;
        a.sum_p -= a.rp[old];
        a.sum_t -= a.rt[old];
        a.count--;
    }
    a.rp[a.head] = p;
    a.rt[a.head] = t;
    a.head = (a.head + 1) % H;
    a.count++;
    a.sum_p += p;
    a.sum_t += t;
}

}  // namespace

extern "C" {

void nba_ipsec_alb_default_params(nba_ipsec_alb_params *p)
{
    if (!p) return;
    p->steps = 25;                    // delta = 4%
    p->init_step = 12;
    p->history = 16384;               // moving-average history
    p->update_ns = 200000000ull;      // update interval 0.2 s
    p->wait_min = 2;                  // waiting interval 2 .. 32 updates
    p->wait_max = 32;
}

int nba_ipsec_alb_create(const nba_ipsec_alb_params *p, nba_ipsec_alb **out)
{
    if (!p || !out) return NBA_IPSEC_EINVAL;
    *out = nullptr;
    if (p->steps == 0 || p->steps > 1000000 || p->init_step > p->steps || p->history == 0 ||
        p->history > (1u << 26) || p->update_ns == 0 || p->wait_max < p->wait_min)
        return NBA_IPSEC_EINVAL;
    nba_ipsec_alb *a = new (std::nothrow) nba_ipsec_alb();
    if (!a) return NBA_IPSEC_ENOMEM;
    try {
        a->rp.assign(p->history, 0);
        a->rt.assign(p->history, 0);
    } catch (...) {
        delete a;
        return NBA_IPSEC_ENOMEM;
    }
    a->p = *p;
    a->k = p->init_step;
    a->dir = +1;
    a->started = false;
    a->waiting = true;
    a->t_end = 0;
    ring_clear(*a);
    a->have_prev = false;
    a->prev_p = a->prev_t = 0;
    a->updates = 0;
    *out = a;
    return NBA_IPSEC_OK;
}

int nba_ipsec_alb_observe(nba_ipsec_alb *a, uint64_t t_ns, uint64_t dt_ns, uint64_t pkts,
                          uint32_t *step)
{
    if (!a) return NBA_IPSEC_EINVAL;
    if (!a->started) {
        // the first sample starts the wait of the initial w
        a->started = true;
        a->waiting = true;
        a->t_end = t_ns + wait_ns(*a, a->k);
    } else if (a->waiting) {
        // L3: the workers are still applying w; samples are discarded
        if (t_ns >= a->t_end) {
            a->waiting = false;
            a->t_end = t_ns + a->p.update_ns;
            ring_clear(*a);
        }
    } else {
        ring_push(*a, pkts, dt_ns);
        if (t_ns >= a->t_end) {
            // L1: compare the moving-average throughput with the previous
            // observation's; P/T < P0/T0  <=>  P*T0 < P0*T
            const unsigned __int128 P = a->sum_p, T = a->sum_t;
            if (a->have_prev && P * a->prev_t < (unsigned __int128)a->prev_p * T)
                a->dir = -a->dir;
            a->have_prev = true;
            a->prev_p = (uint64_t)P;   // <= 2^26 samples x 2^32 packets: fits
            a->prev_t = (uint64_t)T;
            // L5: always move by one step (continuous perturbation); reflect
            // at 0% / 100%
            int64_t k = (int64_t)a->k + a->dir;
            if (k < 0 || k > (int64_t)a->p.steps) {
                a->dir = -a->dir;
                k = (int64_t)a->k + a->dir;
            }
            a->k = (uint32_t)k;
            a->updates++;
            a->waiting = true;
            a->t_end = t_ns + wait_ns(*a, a->k);
        }
    }
    if (step) *step = a->k;
    return NBA_IPSEC_OK;
}

int nba_ipsec_alb_state(const nba_ipsec_alb *a, uint32_t *step, int *direction, uint64_t *updates)
{
    if (!a) return NBA_IPSEC_EINVAL;
    if (step) *step = a->k;
    if (direction) *direction = a->dir;
    if (updates) *updates = a->updates;
    return NBA_IPSEC_OK;
}

int nba_ipsec_alb_destroy(nba_ipsec_alb *a)
{
    delete a;
    return NBA_IPSEC_OK;
}

int nba_ipsec_alb_assign(uint32_t n_sa, uint32_t n_dev, const uint32_t *node_step, uint32_t steps,
                         uint32_t *owner, uint32_t *sa_map)
{
    if (n_dev == 0 || n_dev > NBA_IPSEC_ALB_MAX_DEV || steps == 0 || !owner ||
        (n_dev > 1 && !node_step) || n_sa > (1u << 24))
        return NBA_IPSEC_EINVAL;
    // iterative walk of the tree (L6): node (lo, hi) over SAs [a, b) keeps the
    // first (b - a) - floor((b - a) * step / steps) SAs on [lo, mid)
    struct Node { uint32_t id, lo, hi, a, b; };
    Node stack[2 * NBA_IPSEC_ALB_MAX_DEV];
    int top = 0;
    stack[top++] = {0, 0, n_dev, 0, n_sa};
    while (top > 0) {
        const Node nd = stack[--top];
        if (nd.hi - nd.lo == 1) {
            for (uint32_t s = nd.a; s < nd.b; s++) {
                owner[s] = nd.lo;
                if (sa_map) sa_map[s] = (nd.lo << 24) | s;
            }
            continue;
        }
        if (nd.id >= NBA_IPSEC_ALB_TREE_NODES) return NBA_IPSEC_EINVAL;
        const uint32_t st = node_step[nd.id];
        if (st > steps) return NBA_IPSEC_EINVAL;
        const uint32_t mid = nd.lo + (nd.hi - nd.lo) / 2;
        const uint64_t right = (uint64_t)(nd.b - nd.a) * st / steps;
        const uint32_t cut = nd.b - (uint32_t)right;
        stack[top++] = {2 * nd.id + 1, nd.lo, mid, nd.a, cut};
        stack[top++] = {2 * nd.id + 2, mid, nd.hi, cut, nd.b};
    }
    return NBA_IPSEC_OK;
}

}  // extern "C"
