"""Oracle of the adaptive load balancer -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s baseline legs
may import this module; the product (``libnba_ipsec.so``, ``csrc/alb.cpp``)
shares no code with it.

What it follows: PAPER.md:351-365 (§3.4 "Adaptive CPU/GPU Load Balancing"),
step by step in the paper's order, with the readings L1-L7 of DESIGN.md §2
where the paper is silent:

  * "It chooses the direction (increment or decrement) of the offloading
    fraction w in [0%, 100%] by delta observing if throughput increases or
    decreases"                      -> L1: w = k / K, K = 100% / delta;
    every update moves k by exactly one step; the direction reverses when the
    moving-average throughput of the last observation is LOWER than that of
    the observation before it (equal keeps the direction), and at the ends of
    [0, K] (reflection).
  * "The throughput is measured by the number of packets transmitted out per
    10K CPU cycles.  ... we use the moving average of throughput"
    -> L2: samples are (packets, elapsed ns) per completed batch; the moving
    average over the last `history` samples is sum(packets) / sum(ns); the
    comparison is exact, by cross-multiplication in integers.
  * "let the load balancer wait for all worker threads to apply the updated
    fraction values before next observation and update"
    -> L3: after an update the controller ignores samples for a waiting
    interval, then observes for one update interval (samples before the end of
    the wait are discarded, including the one that ends it).
  * "moving average history size of w to 16384, delta to 4%, and the update
    interval to 0.2 second"          -> defaults.
  * "We also gradually increase the waiting interval from 2 to 32 update
    intervals when we increase w from 0 to 100%"
    -> L4: wait(k) = wait_min + floor((wait_max - wait_min) * k / K) update
    intervals (linear in w).
  * "We continuously insert perturbations (same to delta) to the value of w"
                                      -> L5: there is no "hold"
    state; every update is a move of +-delta, so w keeps probing around the
    optimum and follows it when the workload changes.
  * L6 (B200 target of w): with several devices the split is a binary tree of
    such controllers; node (lo, hi) sends a fraction w of its SAs to its right
    half [mid, hi), mid = lo + (hi - lo) // 2, and the SAs are the node's range
    of SA indices in order (the first n - floor(n * k / K) stay left).
  * L7: a device that owns an SA owns its sequence counter; when ownership
    moves, the counter moves with it (the gateway's output is unchanged).

Parity status: pinned by tests/test_alb.py (hand-derived trajectories,
convergence on closed-form throughput curves, assignment invariants).
"""
from __future__ import annotations

from collections import deque


class Controller:
    """One hill-climbing controller, plain Python."""

    def __init__(self, steps=25, init_step=None, history=16384, update_ns=200_000_000,
                 wait_min=2, wait_max=32):
        self.K = int(steps)
        self.k = self.K // 2 if init_step is None else int(init_step)
        self.H = int(history)
        self.U = int(update_ns)
        self.wmin, self.wmax = int(wait_min), int(wait_max)
        self.dir = +1
        self.started = False
        self.waiting = True
        self.t_end = 0
        self.ring = deque()
        self.prev = None          # (packets, ns) of the previous observation
        self.updates = 0

    def wait_intervals(self, k):
        # L4: linear from wait_min at w = 0 to wait_max at w = 100%
        return self.wmin + (self.wmax - self.wmin) * k // self.K

    def observe(self, t_ns, dt_ns, pkts):
        """Feed one completed batch (clock t_ns, its duration dt_ns, packets
        transmitted); returns the step k (w = k / K) to apply from now on."""
        if not self.started:                       # the first call starts a wait
            self.started = True
            self.waiting = True
            self.t_end = t_ns + self.wait_intervals(self.k) * self.U
            return self.k
        if self.waiting:                           # L3: workers still applying w
            if t_ns >= self.t_end:
                self.waiting = False
                self.t_end = t_ns + self.U
                self.ring.clear()
            return self.k
        self.ring.append((int(pkts), int(dt_ns)))  # L2: moving-average window
        if len(self.ring) > self.H:
            self.ring.popleft()
        if t_ns < self.t_end:
            return self.k
        P = sum(p for p, _ in self.ring)
        T = sum(d for _, d in self.ring)
        if self.prev is not None:
            P0, T0 = self.prev
            if P * T0 < P0 * T:                   # throughput decreased: reverse (L1)
                self.dir = -self.dir
        self.prev = (P, T)
        k = self.k + self.dir
        if k < 0 or k > self.K:                    # reflect at the ends of [0, 100%]
            self.dir = -self.dir
            k = self.k + self.dir
        self.k = k
        self.updates += 1
        self.waiting = True
        self.t_end = t_ns + self.wait_intervals(self.k) * self.U
        return self.k


def assign(n_sa, n_dev, node_step, steps):
    """Owner device of every SA under the binary tree of splits (L6).
    node_step[i] is the step of heap node i (root 0, children 2i+1 / 2i+2)."""
    owner = [0] * n_sa

    def rec(node, lo, hi, a, b):
        if hi - lo == 1:
            for s in range(a, b):
                owner[s] = lo
            return
        mid = lo + (hi - lo) // 2
        n = b - a
        n_right = n * node_step[node] // steps
        cut = b - n_right
        rec(2 * node + 1, lo, mid, a, cut)
        rec(2 * node + 2, mid, hi, cut, b)

    if n_dev >= 1:
        rec(0, 0, n_dev, 0, n_sa)
    return owner
