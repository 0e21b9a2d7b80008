"""Adaptive load balancer.

Pins of the oracle (oracle/alb.py) against what the paper and arithmetic fix
-- a hand-derived trajectory, the closed-form schedule of the waiting
intervals (L4), convergence to the argmax of a closed-form throughput curve and
tracking of a moved optimum (L1, L5), reflection at the ends, and the owner map
(L6) against its closed form for two devices -- then parity of the library's
controller and assignment (csrc/alb.cpp through the C ABI; host code, no GPU)
with the oracle on seeded sample streams."""
import ctypes

import numpy as np
import pytest

from oracle import alb as oalb
from paper_conf_eurosys_kimjlmsm15_b200 import alb, nba_ipsec


def _drive(ctl, samples):
    return [ctl.observe(t, dt, p) for t, dt, p in samples]


# ---- oracle pins --------------------------------------------------------------

HAND = dict(steps=4, init_step=2, history=100, update_ns=10, wait_min=1, wait_max=1)
# (t, dt, packets) and the step after each call, derived by hand from
# PAPER.md:355-359 under L1-L5: start -> wait 10 ns -> observe 10 ns -> move.
HAND_SAMPLES = [(0, 0, 0), (5, 5, 50), (10, 5, 50), (15, 5, 50), (20, 5, 50),   # no previous: +1
                (30, 10, 0), (40, 10, 80),        # 8/ns < 10/ns: reverse, 3 -> 2
                (50, 10, 0), (60, 10, 90),        # 9 > 8: keep, 2 -> 1
                (70, 10, 0), (80, 10, 90),        # equal: keep, 1 -> 0
                (90, 10, 0), (100, 10, 100)]      # up, keep -1 -> -1 reflects to 1
HAND_STEPS = [2, 2, 2, 2, 3, 3, 2, 2, 1, 1, 0, 0, 1]


def test_oracle_hand_trajectory():
    assert _drive(oalb.Controller(**HAND), HAND_SAMPLES) == HAND_STEPS


def test_oracle_wait_schedule_closed_form():
    # constant throughput never reverses, so w climbs one step per update and
    # update j+1 happens (wait(k_{j+1}) + 1) update intervals after update j
    U, K = 100, 25
    c = oalb.Controller(steps=K, init_step=0, history=1000, update_ns=U, wait_min=2, wait_max=32)
    times, last = [], c.k
    for t in range(0, 40000):
        k = c.observe(t, 1, 7)
        if k != last:
            times.append(t)
            last = k
    expect, t, k = [], 0, 0
    t = (2 + 30 * 0 // K) * U + U            # first wait (w = 0) + one observation
    while t < 40000 and k < K:
        expect.append(t)
        k += 1
        t += (2 + 30 * k // K) * U + U
    assert times[:len(expect)] == expect
    assert [2 + 30 * k // K for k in (0, 12, 25)] == [2, 16, 32]     # L4 end points


def _two_device_sim(ctl, rates_fn, n_updates, N=100_000, jitter=0.0, seed=0):
    """Two devices run a step's share concurrently: the right one gets
    floor(N k / K) packets; step time = max over devices (integer ns)."""
    rng = np.random.default_rng(seed)
    t, ks = 0, []
    K = ctl.K
    while ctl.updates < n_updates:
        r0, r1 = rates_fn(ctl.updates)
        nr = N * ctl.k // K
        dt = max(-(-(N - nr) // r0), -(-nr // r1), 1)
        if jitter:
            dt = int(dt * (1.0 + jitter * rng.standard_normal()))
        t += dt
        before = ctl.updates
        ctl.observe(t, dt, N)
        if ctl.updates != before:
            ks.append(ctl.k)
    return ks


def _best_k(r0, r1, K=25, N=100_000):
    return int(np.argmax([N / max(-(-(N - N * k // K) // r0), -(-(N * k // K) // r1), 1)
                          for k in range(K + 1)]))


@pytest.mark.parametrize("jitter", [0.0, 0.01])
def test_oracle_converges_and_tracks(jitter):
    U = 2_000_000
    c = oalb.Controller(steps=25, init_step=12, history=64, update_ns=U, wait_min=2, wait_max=8)
    # device 0 three times as fast as device 1, then the reverse (L5 tracking)
    rates = lambda j: (300, 100) if j < 60 else (100, 300)       # noqa: E731
    ks = _two_device_sim(c, rates, 120, jitter=jitter, seed=3)
    k1, k2 = _best_k(300, 100), _best_k(100, 300)
    assert (k1, k2) == (6, 19)
    tail1, tail2 = np.array(ks[30:60]), np.array(ks[100:120])
    assert abs(tail1.mean() - k1) <= 1.0 and tail1.min() >= k1 - 2 and tail1.max() <= k1 + 2
    assert abs(tail2.mean() - k2) <= 1.0 and tail2.min() >= k2 - 2 and tail2.max() <= k2 + 2


def test_oracle_reflects_at_the_ends():
    # throughput grows with w: w reaches 100% and then probes K-1, K, K-1, ...
    c = oalb.Controller(steps=5, init_step=3, history=8, update_ns=50, wait_min=1, wait_max=1)
    ks = _two_device_sim(c, lambda j: (1, 10_000), 12, N=10_000)
    assert ks[:2] == [4, 5] and set(ks[2:]) <= {4, 5} and 5 in ks[2:] and 4 in ks[2:]


@pytest.mark.parametrize("n_sa", [0, 1, 7, 1024])
def test_oracle_assign_two_devices_closed_form(n_sa):
    K = 25
    for k in range(K + 1):
        owner = oalb.assign(n_sa, 2, [k], K)
        cut = n_sa - n_sa * k // K
        assert owner == [0] * cut + [1] * (n_sa - cut)


def test_oracle_assign_tree_invariants():
    rng = np.random.default_rng(5)
    for n_dev in range(1, 9):
        for _ in range(20):
            n_sa = int(rng.integers(0, 3000))
            K = int(rng.choice([4, 25, 100]))
            st = [int(x) for x in rng.integers(0, K + 1, 15)]
            owner = oalb.assign(n_sa, n_dev, st, K)
            assert len(owner) == n_sa and all(0 <= o < n_dev for o in owner)
            assert all(a <= b for a, b in zip(owner, owner[1:]))   # contiguous, device order
        assert set(oalb.assign(64, n_dev, [0] * 15, 25)) == {0}
        assert set(oalb.assign(64, n_dev, [25] * 15, 25)) == {n_dev - 1}
    # balanced tree with w = 1/2 everywhere splits 1024 SAs evenly over 8 devices
    assert np.bincount(oalb.assign(1024, 8, [2] * 15, 4)).tolist() == [128] * 8


# ---- library (csrc/alb.cpp) vs oracle ------------------------------------------

def _random_stream(rng, n):
    t = 0
    out = []
    for _ in range(n):
        dt = int(rng.integers(1, 2000))
        t += dt if rng.random() > 0.05 else 0          # repeated clock values
        out.append((t, dt, int(rng.integers(0, 70_000))))
    return out


@pytest.mark.parametrize("seed", range(6))
def test_library_controller_matches_oracle(seed):
    rng = np.random.default_rng([41, seed])
    K = int(rng.choice([1, 4, 25, 100]))
    prm = dict(steps=K, init_step=int(rng.integers(0, K + 1)), history=int(rng.choice([1, 3, 64])),
               update_ns=int(rng.integers(500, 20_000)), wait_min=int(rng.integers(0, 3)),
               wait_max=int(rng.integers(3, 9)))
    s = _random_stream(rng, 6000)
    lib_c = nba_ipsec.Alb(**prm)
    got = _drive(lib_c, s)
    want = _drive(oalb.Controller(**prm), s)
    assert got == want
    assert lib_c.state()[2] > 5                      # the stream did move w


def test_library_hand_trajectory_and_defaults():
    assert _drive(nba_ipsec.Alb(**HAND), HAND_SAMPLES) == HAND_STEPS
    p = nba_ipsec.alb_default_params()
    assert (p.steps, p.history, p.update_ns, p.wait_min, p.wait_max) == (25, 16384, 200_000_000, 2, 32)


def test_library_converges_like_oracle():
    prm = dict(steps=25, init_step=12, history=64, update_ns=2_000_000, wait_min=2, wait_max=8)
    rates = lambda j: (300, 100) if j < 40 else (100, 300)       # noqa: E731

    class Wrap:                                      # the simulation reads k / K / updates
        def __init__(self):
            self.c = nba_ipsec.Alb(**prm)
            self.K = 25

        @property
        def k(self):
            return self.c.state()[0]

        @property
        def updates(self):
            return self.c.state()[2]

        def observe(self, *a):
            return self.c.observe(*a)

    a = _two_device_sim(Wrap(), rates, 60, jitter=0.01, seed=9)
    b = _two_device_sim(oalb.Controller(**prm), rates, 60, jitter=0.01, seed=9)
    assert a == b


def test_library_assign_matches_oracle():
    rng = np.random.default_rng(17)
    for n_dev in range(1, 9):
        for _ in range(10):
            n_sa = int(rng.integers(0, 5000))
            K = int(rng.choice([1, 4, 25, 1000]))
            st = rng.integers(0, K + 1, 15).astype(np.uint32)
            owner, sa_map = nba_ipsec.alb_assign(n_sa, n_dev, st, K)
            assert owner.tolist() == oalb.assign(n_sa, n_dev, st.tolist(), K)
            assert np.array_equal(sa_map >> 24, owner)
            assert np.array_equal(sa_map & 0xFFFFFF, np.arange(n_sa))


def test_library_alb_argument_errors():
    L = nba_ipsec.lib
    h = ctypes.c_void_p()
    for bad in (dict(steps=0), dict(steps=4, init_step=5), dict(history=0), dict(update_ns=0),
                dict(wait_min=5, wait_max=4)):
        p = nba_ipsec.alb_default_params()
        for k, v in bad.items():
            setattr(p, k, v)
        assert L.nba_ipsec_alb_create(ctypes.byref(p), ctypes.byref(h)) == nba_ipsec.EINVAL
    assert L.nba_ipsec_alb_observe(None, 0, 0, 0, None) == nba_ipsec.EINVAL
    assert L.nba_ipsec_alb_destroy(None) == nba_ipsec.OK
    u32p = ctypes.POINTER(ctypes.c_uint32)
    own = (ctypes.c_uint32 * 4)()
    st = (ctypes.c_uint32 * 15)(*([3] * 15))
    assert L.nba_ipsec_alb_assign(4, 0, st, 25, own, None) == nba_ipsec.EINVAL
    assert L.nba_ipsec_alb_assign(4, 9, st, 25, own, None) == nba_ipsec.EINVAL
    assert L.nba_ipsec_alb_assign(4, 2, st, 2, own, None) == nba_ipsec.EINVAL    # step > steps
    assert L.nba_ipsec_alb_assign(4, 2, None, 25, own, None) == nba_ipsec.EINVAL
    assert L.nba_ipsec_alb_assign(4, 1, None, 25, own, None) == nba_ipsec.OK
    assert L.nba_ipsec_alb_assign(4, 2, st, 25, ctypes.cast(None, u32p), None) == nba_ipsec.EINVAL


def test_balancer_tree_feeds_subtrees():
    # 4 devices: root splits {0,1} | {2,3}; each node sees its subtree's packets
    # and slowest device
    b = alb.Balancer(64, 4, steps=4, init_step=2, history=10, update_ns=10, wait_min=1, wait_max=1)
    assert [n for n, _, _ in b.nodes] == [0, 1, 2]
    owner, _ = b.assignment()
    assert np.bincount(owner).tolist() == [16] * 4
    t = 0
    for j in range(6):
        t += 10
        # device 3 is slow: node 2 ({2,3}) sees its throughput fall as w moves right
        b.observe(t, [10, 10, 10, 10 + 30 * (j > 2)], [100, 100, 100, 100])
    assert b.ctl[0].state()[2] >= 1 and b.ctl[2].state()[2] >= 1
