"""The benchmark's exact timed path against the oracle ("GPU vs
oracle: memcmp of every slot ... on all configs"; §4.1).

bench.py times the software-pipelined persistent ring (k_fused_ring_pipe)
over R device copies of one full-size batch (65,536 packets, 1024 SAs; R from
device.ring_slot_count, the bench's own formula), every timed batch through
nba_ipsec_ring_run_batches.  Here the same ring runs 2R + 5 batches (two
rotations and a partial one), then a second run continues mid-rotation from
the cursor, with and without per-batch timestamps.  The oracle runs the same
batch sequence with carried SA state; each slot's WHOLE output pool must equal
the oracle's output of the last batch that used that slot, and out_len, the
final SA counters and the device counters must match.  The C5 sweep sizes
(configs[4]: 128 / 256 / 512 / 1024 B) run the same way with R + 3 batches."""
import numpy as np
import pytest

import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen, shard

pytestmark = pytest.mark.gpu

N_PKTS = 65536
N_SA = 1024


def _ring_vs_oracle(size, cfg_id, runs, timestamps=False, form=None):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    p, b = shard.rank_workload(cfg_id, N_PKTS, size, N_SA, 0, 1)
    l2 = int(torch.cuda.get_device_properties(0).L2_cache_size)
    R = device.ring_slot_count(b.in_len, b.n, l2)
    sas = oracle.make_sas(p)
    ctr = oracle.Counters()
    with nba_ipsec.SATable(p, device=0, max_batch=N_PKTS) as t:
        d0 = device.to_device(b, "cuda")
        dbs = [d0] + [device.clone(d0) for _ in range(R - 1)]
        ring = t.ring([(*d.args(), b.n) for d in dbs])
        if form is not None:
            ring.set_form(form)
        expect_form = form if form is not None else nba_ipsec.Ring.PIPELINED
        assert ring.form == expect_form
        ts = None
        if timestamps:
            ts = torch.zeros(max(runs) + 1, dtype=torch.int64, device="cuda")
            ring.set_timestamps(ts)
        last = {}                       # slot -> (out pool, out_len) of its last batch
        k = 0
        for nb in runs:
            ring.run_batches(nb)
            for _ in range(nb):
                out, ol, _ = oracle.process_batch(sas, N_SA, b, n_threads=16, counters=ctr)
                last[k % R] = (out, ol.copy())
                k += 1
            if ts is not None:
                torch.cuda.synchronize()
                v = ts[:nb + 1].cpu().numpy()
                assert np.all(v > 0) and np.all(np.diff(v) >= 0), "per-batch stamps not monotone"
        torch.cuda.synchronize()
        assert ring.cursor == k % R
        for s, (o_out, o_len) in last.items():
            g_out, g_len = device.fetch(dbs[s])
            assert np.array_equal(g_len, o_len), f"slot {s}: out_len differs"
            if not np.array_equal(g_out, o_out):
                d = np.nonzero(g_out != o_out)[0]
                raise AssertionError(f"slot {s}: {d.size} output-pool bytes differ, first at {d[:8]}")
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, N_SA)), "final SA counters differ"
        assert t.counters() == ctr.as_dict()
        ring.close()
    return R


@pytest.mark.parametrize("cfg_id,size", [(2, 64), (3, 1514), (4, "imix")])
def test_bench_ring_exact(cfg_id, size):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device
    p, b = shard.rank_workload(cfg_id, N_PKTS, size, N_SA, 0, 1)
    R = device.ring_slot_count(b.in_len, b.n, int(torch.cuda.get_device_properties(0).L2_cache_size))
    _ring_vs_oracle(size, cfg_id, [2 * R + 5, max(1, R - 2)], timestamps=(cfg_id == 2))


@pytest.mark.parametrize("size", [128, 256, 512, 1024])
def test_sweep_sizes_ring(size):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device
    p, b = shard.rank_workload(5, N_PKTS, size, N_SA, 0, 1)
    R = device.ring_slot_count(b.in_len, b.n, int(torch.cuda.get_device_properties(0).L2_cache_size))
    _ring_vs_oracle(size, 5, [R + 3])


def test_bench_ring_plain_persistent_form():
    """The plain persistent form (set_form) over the same full-size 64-B ring."""
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    _ring_vs_oracle(64, 2, [7, 9], form=nba_ipsec.Ring.PERSISTENT)


@pytest.mark.parametrize("size", [128, 256, 512, 1024])
def test_sweep_sizes_process_batch(size):
    """configs[4] sizes at full size through process_batch, 3 batches."""
    from harness import assert_same, gpu_run, oracle_run
    p, b = shard.rank_workload(5, N_PKTS, size, N_SA, 0, 1)
    batches = [b, gen.make_batch(N_PKTS, size, N_SA, cfg_id=5, batch=1), b]
    assert_same(gpu_run(p, batches), oracle_run(p, batches, n_threads=16))
