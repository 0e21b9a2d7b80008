"""The benchmark's exact timed path against the oracle ("GPU vs
oracle: memcmp of every slot ... on all configs"; §4.1).

bench.py times the batch ring's default form (the role-split ring
k_fused_ring_roles -- sorted mode at IMIX -- except the software-pipelined
k_fused_ring_pipe at 1514 B; each also run in the other form here) over R device copies of one full-size batch (65,536 packets, 1024 SAs; R from
device.ring_slot_count, the bench's own formula), every timed batch through
nba_ipsec_ring_run_batches.  Here the same ring runs 2R + 5 batches (two
rotations and a partial one), then a second run continues mid-rotation from
the cursor, with and without per-batch timestamps.  The oracle runs the same
batch sequence with carried SA state; each slot's WHOLE output pool must equal
the oracle's output of the last batch that used that slot, and out_len, the
final SA counters and the device counters must match.  The C5 sweep sizes
(configs[4]: 128 / 256 / 512 / 1024 B) run the same way with R + 3 batches.
The bench's inbound protocol (R ESP batches through an inbound ring, windows
reset per rotation) runs against the oracle's sequential receiver the same
way, at 64 B (software-pipelined inbound ring) and IMIX (graph ring)."""
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
        # default: the role-split form for one-length rings of frames up to 1024 B
        # and for mixed rings of more than 4 slots (IMIX: R = 7, sorted mode),
        # else the pipelined one
        expect_form = form if form is not None else (
            nba_ipsec.Ring.PIPELINED if size == 1514 else nba_ipsec.Ring.ROLES)
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


@pytest.mark.parametrize("cfg_id,size", [(2, 64), (3, 1514), (4, "imix")])
def test_bench_ring_free_form(cfg_id, size):
    """The free-running-lanes form (k_fused_ring_free, set_form) over the same
    full-size ring: two rotations and a partial one, then a run continuing
    mid-rotation, against the oracle."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    p, b = shard.rank_workload(cfg_id, N_PKTS, size, N_SA, 0, 1)
    R = device.ring_slot_count(b.in_len, b.n, int(torch.cuda.get_device_properties(0).L2_cache_size))
    _ring_vs_oracle(size, cfg_id, [2 * R + 5, max(1, R - 2)], timestamps=(cfg_id == 4),
                    form=nba_ipsec.Ring.FREE)


@pytest.mark.parametrize("cfg_id,size", [(2, 64), (5, 256), (4, "imix")])
def test_bench_ring_pipelined_form(cfg_id, size):
    """The software-pipelined form (set_form; the default before the role-split
    form) over the same full-size one-length rings, against the oracle."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    p, b = shard.rank_workload(cfg_id, N_PKTS, size, N_SA, 0, 1)
    R = device.ring_slot_count(b.in_len, b.n, int(torch.cuda.get_device_properties(0).L2_cache_size))
    _ring_vs_oracle(size, cfg_id, [2 * R + 5, max(1, R - 2)], timestamps=(cfg_id == 2),
                    form=nba_ipsec.Ring.PIPELINED)


@pytest.mark.parametrize("cfg_id,size", [(3, 1514)])
def test_bench_ring_roles_form(cfg_id, size):
    """The role-split form (set_form) over the full-size 1514-B ring: two
    rotations and a partial one, then a run continuing mid-rotation, with
    timestamps."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    p, b = shard.rank_workload(cfg_id, N_PKTS, size, N_SA, 0, 1)
    R = device.ring_slot_count(b.in_len, b.n, int(torch.cuda.get_device_properties(0).L2_cache_size))
    _ring_vs_oracle(size, cfg_id, [2 * R + 5, max(1, R - 2)], timestamps=True, form=nba_ipsec.Ring.ROLES)


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


def _inbound_compare(ds, sts, last, tag):
    from paper_conf_eurosys_kimjlmsm15_b200 import device
    for s, (o_out, o_len, o_st, ib) in last.items():
        g_out, g_len = device.fetch(ds[s])
        assert np.array_equal(sts[s].cpu().numpy(), o_st), f"{tag} slot {s}: status differs"
        assert np.array_equal(g_len, o_len), f"{tag} slot {s}: out_len differs"
        mask = np.zeros(o_out.size, bool)
        for i in np.nonzero(o_len)[0]:
            a = int(ib.out_off[i])
            mask[a:a + int(o_len[i])] = True
        if not np.array_equal(g_out[:o_out.size][mask], o_out[mask]):
            raise AssertionError(f"{tag} slot {s}: inner bytes differ")


@pytest.mark.parametrize("cfg_id,size,form", [(2, 64, "pipelined"), (4, "imix", "graph")])
def test_bench_inbound_ring_exact(cfg_id, size, form):
    """bench.py's inbound protocol at full size against the oracle's sequential
    receiver: R ESP batches from R consecutive outbound batches (the oracle's
    output, with carried SA counters), an inbound ring over them in the form
    the library picks by length (64 B: the software-pipelined ring; IMIX: the
    graph ring); one rotation after reset_inbound (every packet accepted), then
    three batches without a reset (every packet a replay).  Every slot's
    statuses, out_len and the inner bytes of every accepted packet, the
    windows and the counters equal the oracle's (RFC 4303 §3.4)."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    p, b = shard.rank_workload(cfg_id, N_PKTS, size, N_SA, 0, 1)
    R = device.ring_slot_count(b.in_len, b.n, int(torch.cuda.get_device_properties(0).L2_cache_size))
    sas = oracle.make_sas(p)
    esp = []
    for _ in range(R):
        out, ol, _ = oracle.process_batch(sas, N_SA, b, n_threads=16)
        esp.append(gen.Batch(n=b.n, in_buf=out, in_off=b.out_off.copy(), in_len=ol.copy(),
                             sa_idx=b.sa_idx.copy(), out_off=b.out_off.copy(),
                             out_pool_bytes=b.out_pool_bytes, frame_len=b.frame_len))
    sas_in = oracle.make_sas(p)
    ctr = oracle.InCounters()
    with nba_ipsec.SATable(p, device=0, max_batch=N_PKTS) as t:
        t.enable_inbound()
        ds = [device.to_device(e, "cuda", out_fill=0xA5) for e in esp]
        sts = [torch.full((b.n,), 0xff, dtype=torch.uint8, device="cuda") for _ in esp]
        ring = t.ring_inbound([(*d.args(), st, e.n) for d, st, e in zip(ds, sts, esp)])
        assert ring.form == {"graph": ring.GRAPH, "pipelined": ring.PIPELINED}[form]
        # a rotation from fresh windows
        t.reset_inbound()
        ring.run_batches(R)
        win = oracle.make_windows(oracle.make_sas(p), N_SA)
        last = {}
        for k in range(R):
            o_out, o_len, o_st, _ = oracle.process_inbound(sas_in, win, N_SA, esp[k], counters=ctr)
            assert np.all(o_st == 0)
            last[k] = (o_out, o_len.copy(), o_st.copy(), esp[k])
        torch.cuda.synchronize()
        _inbound_compare(ds, sts, last, "rotation")
        # three more batches, no reset: replays
        ring.run_batches(3)
        last = {}
        for k in range(3):
            o_out, o_len, o_st, _ = oracle.process_inbound(sas_in, win, N_SA, esp[k], counters=ctr)
            assert np.all(o_st == 3)
            last[k] = (o_out, o_len.copy(), o_st.copy(), esp[k])
        torch.cuda.synchronize()
        _inbound_compare(ds, sts, last, "replays")
        top, bmp = t.replay_window()
        o_top, o_bmp = oracle.window_state(win, N_SA)
        assert np.array_equal(top, o_top) and np.array_equal(bmp, o_bmp)
        assert t.in_counters() == ctr.as_dict()
        ring.close()
