"""GPU parity for batch rings (nba_ipsec_ring_*): a fixed set of batch slots
recorded as one CUDA graph and replayed must give exactly what the same
sequence of process_batch calls gives -- here against the oracle processing
the slots' batches in ring order, round after round (the slots are refilled
between runs, in stream order), including the final SA counters and the
device counters; and replay equals stream launches on a second table."""
import numpy as np
import pytest

import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen

pytestmark = pytest.mark.gpu


def _slot(db):
    return (db.in_buf, db.in_off, db.in_len, db.sa_idx, db.out_buf, db.out_off, db.out_len, db.n)


@pytest.mark.parametrize("pipe", [False, True])
@pytest.mark.parametrize("sizes,n_sa", [((64, "imix", 1514), 1024), (("imix", "imix"), 7)])
def test_ring_rounds_match_oracle(sizes, n_sa, pipe, monkeypatch):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    if not pipe:     # the plain persistent form (default: software-pipelined)
        monkeypatch.setenv("NBA_IPSEC_RING_NOPIPE", "1")
    p = gen.make_sas(n_sa, cfg_id=51)
    n = 20000
    sas = oracle.make_sas(p)
    ctr = oracle.Counters()
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        dbs = [device.to_device(gen.make_batch(n, s, n_sa, cfg_id=51, batch=i), "cuda")
               for i, s in enumerate(sizes)]
        ring = t.ring([_slot(d) for d in dbs])
        for rnd in range(3):
            # refill the slots with this round's traffic (stream order), run one pass
            hb = [gen.make_batch(n, s, n_sa, cfg_id=51, batch=100 * rnd + i)
                  for i, s in enumerate(sizes)]
            hb[0].sa_idx[::97] = n_sa + 1                      # some invalid SAs
            for d, b in zip(dbs, hb):
                d.in_buf.copy_(torch.from_numpy(b.in_buf))
                d.in_len.copy_(torch.from_numpy(b.in_len.view(np.int16)))
                d.sa_idx.copy_(torch.from_numpy(b.sa_idx.view(np.int32)))
            ring.run(1)
            torch.cuda.synchronize()
            for d, b in zip(dbs, hb):
                o_out, o_len, _ = oracle.process_batch(sas, n_sa, b, n_threads=8, counters=ctr)
                g_out, g_len = device.fetch(d)
                assert np.array_equal(g_len, o_len)
                for i in np.nonzero(o_len)[0][::7]:
                    a, L = int(b.out_off[i]), int(o_len[i])
                    assert np.array_equal(g_out[a:a + L], o_out[a:a + L])
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa))
        assert t.counters() == ctr.as_dict()
        ring.close()


@pytest.mark.parametrize("pipe", [False, True])
def test_ring_replay_equals_stream_launches(pipe, monkeypatch):
    import torch
    if not pipe:
        monkeypatch.setenv("NBA_IPSEC_RING_NOPIPE", "1")
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    p = gen.make_sas(1024, cfg_id=52)
    b = gen.make_batch(65536, 64, 1024, cfg_id=52)
    da = [device.to_device(b, "cuda") for _ in range(3)]
    db_ = [device.to_device(b, "cuda") for _ in range(3)]
    with nba_ipsec.SATable(p, device=0, max_batch=b.n) as ta, \
            nba_ipsec.SATable(p, device=0, max_batch=b.n) as tb:
        ring = ta.ring([_slot(d) for d in da])
        s = torch.cuda.Stream()
        ring.run(4, stream=s)
        s.synchronize()
        for _ in range(4):
            for d in db_:
                tb.process(*d.args(), n=b.n)
        torch.cuda.synchronize()
        for x, y in zip(da, db_):
            assert torch.equal(x.out_buf, y.out_buf) and torch.equal(x.out_len, y.out_len)
        assert np.array_equal(ta.sa_seq(), tb.sa_seq())
        assert ta.counters() == tb.counters()
        ring.close()


def test_ring_rejects_bad_slots():
    import ctypes
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    p = gen.make_sas(4, cfg_id=53)
    with nba_ipsec.SATable(p, device=0, max_batch=100) as t:
        h = ctypes.c_void_p()
        bad = (nba_ipsec.Batch * 1)()
        bad[0] = nba_ipsec.Batch(0, 0, 0, 0, 0, 0, 0, 50)     # NULL buffers
        assert nba_ipsec.lib.nba_ipsec_ring_create(t._h, bad, 1, ctypes.byref(h)) == nba_ipsec.EINVAL
        assert nba_ipsec.lib.nba_ipsec_ring_create(t._h, bad, 0, ctypes.byref(h)) == nba_ipsec.EINVAL
        assert nba_ipsec.lib.nba_ipsec_ring_destroy(None) == nba_ipsec.OK


@pytest.mark.parametrize("n,pipeline", [(100_000, None), (30_000, 1)])
def test_ring_two_kernel_and_unfused_paths(n, pipeline):
    """Batches larger than one super-round per CTA take the two-kernel path
    (prologue + fused, chained by programmatic dependent launch); the unfused
    pipeline launches five kernels: both recorded in the ring's graph must still
    equal the oracle over rounds."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa = 1024
    p = gen.make_sas(n_sa, cfg_id=54)
    b = gen.make_batch(n, "imix", n_sa, cfg_id=54)
    sas = oracle.make_sas(p)
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        if pipeline is not None:
            t.set_pipeline(pipeline)
        d = device.to_device(b, "cuda")
        ring = t.ring([_slot(d)])
        ring.run(2)
        torch.cuda.synchronize()
        oracle.process_batch(sas, n_sa, b, n_threads=8)
        o_out, o_len, _ = oracle.process_batch(sas, n_sa, b, n_threads=8)
        g_out, g_len = device.fetch(d)
        assert np.array_equal(g_len, o_len)
        assert np.array_equal(g_out, o_out)
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa))
        ring.close()


@pytest.mark.parametrize("form", ["graph", "persistent", "pipelined"])
def test_inbound_ring_equals_stream_launches_and_oracle(form, monkeypatch):
    """ESP inbound slots in a ring (graph form, the opt-in plain persistent form
    and the software-pipelined form, each forced): status, inner bytes, lengths,
    windows and counters equal process_inbound from the stream and the
    oracle's receiver."""
    import torch
    if form == "graph":
        monkeypatch.setenv("NBA_IPSEC_RING_IN_PIPE", "0")
    if form == "persistent":
        monkeypatch.setenv("NBA_IPSEC_RING_IN_PERSIST", "1")
    if form == "pipelined":
        monkeypatch.setenv("NBA_IPSEC_RING_IN_PIPE", "1")
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa, n = 64, 5000
    p = gen.make_sas(n_sa, cfg_id=55)
    sas = oracle.make_sas(p)
    win = oracle.make_windows(sas, n_sa)
    esp = []
    for j in range(3):                                   # three consecutive outbound batches
        b = gen.make_batch(n, "imix", n_sa, cfg_id=55, batch=j)
        e_out, e_len, _ = oracle.process_batch(sas, n_sa, b)
        ib = gen.esp_batch(e_out, b.out_off, e_len, b.sa_idx, np.arange(n))
        esp.append(ib)
    sas_in = oracle.make_sas(p)
    ref = [oracle.process_inbound(sas_in, win, n_sa, ib) for ib in esp]
    with nba_ipsec.SATable(p, device=0, max_batch=n) as ta, \
            nba_ipsec.SATable(p, device=0, max_batch=n) as tb:
        ta.enable_inbound()
        tb.enable_inbound()
        da = [device.to_device(ib, "cuda") for ib in esp]
        db_ = [device.to_device(ib, "cuda") for ib in esp]
        sa_ = [torch.zeros(ib.n, dtype=torch.uint8, device="cuda") for ib in esp]
        sb_ = [torch.zeros(ib.n, dtype=torch.uint8, device="cuda") for ib in esp]
        ring = ta.ring_inbound([(*d.args(), st, ib.n) for d, st, ib in zip(da, sa_, esp)])
        assert ring.form == {"graph": ring.GRAPH, "persistent": ring.PERSISTENT,
                             "pipelined": ring.PIPELINED}[form]
        ring.run(1)
        for d, st, ib in zip(db_, sb_, esp):
            tb.process_inbound(*d.args(), status=st, n=ib.n)
        torch.cuda.synchronize()
        for k, (ib, (o_out, o_len, o_st, _)) in enumerate(zip(esp, ref)):
            ga, la = device.fetch(da[k])
            gb, lb = device.fetch(db_[k])
            assert np.array_equal(sa_[k].cpu().numpy(), o_st) and np.array_equal(sb_[k].cpu().numpy(), o_st)
            assert np.array_equal(la, o_len) and np.array_equal(lb, o_len)
            for i in np.nonzero(o_len)[0][::5]:
                a, L = int(ib.out_off[i]), int(o_len[i])
                assert np.array_equal(ga[a:a + L], o_out[a:a + L])
        ta_top, ta_bmp = ta.replay_window()
        o_top, o_bmp = oracle.window_state(win, n_sa)
        assert np.array_equal(ta_top, o_top) and np.array_equal(ta_bmp, o_bmp)
        assert ta.in_counters() == tb.in_counters()
        ring.close()


@pytest.mark.parametrize("force_graph", [False, True])
def test_ring_flow_table_slots_persistent_and_graph(force_graph, monkeypatch):
    """Slots without SA indices (the one-kernel path looks each packet's SA up in
    the flow table) in a ring -- the persistent form (one launch walks all
    batches) and, forced, the graph form -- equal the oracle over 3 rounds."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    if force_graph:
        monkeypatch.setenv("NBA_IPSEC_RING_GRAPH", "1")
    else:
        monkeypatch.delenv("NBA_IPSEC_RING_GRAPH", raising=False)
    n_sa, n = 256, 30000
    p = gen.make_sas(n_sa, cfg_id=56)
    f = gen.make_flows(3000, n_sa, cfg_id=56)
    bs = []
    for k in range(2):
        b = gen.make_batch(n, "imix", n_sa, cfg_id=56, batch=k)
        gen.apply_flows(b, f, cfg_id=56, batch=k, miss=0.05)
        b.sa_idx = oracle.flow_lookup(f, b)
        bs.append(b)
    sas = oracle.make_sas(p)
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        t.set_flow_table(f)
        ds = [device.to_device(b, "cuda") for b in bs]
        ring = t.ring([(d.in_buf, d.in_off, d.in_len, None, d.out_buf, d.out_off, d.out_len, n)
                       for d in ds])
        ring.run(3)
        torch.cuda.synchronize()
        for _ in range(2):
            for b in bs:
                oracle.process_batch(sas, n_sa, b, n_threads=8)
        for d, b in zip(ds, bs):
            o_out, o_len, _ = oracle.process_batch(sas, n_sa, b, n_threads=8)
            g_out, g_len = device.fetch(d)
            assert np.array_equal(g_len, o_len) and np.array_equal(g_out, o_out)
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa))
        ring.close()


def test_ring_refuses_after_flow_table_replaced():
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa, n = 16, 1000
    p = gen.make_sas(n_sa, cfg_id=57)
    b = gen.make_batch(n, 64, n_sa, cfg_id=57)
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        t.set_flow_table(gen.make_flows(100, n_sa, cfg_id=57))
        d = device.to_device(b, "cuda")
        ring = t.ring([(*d.args(), n)])
        ring.run(1)
        t.set_flow_table(gen.make_flows(200, n_sa, cfg_id=58))
        with pytest.raises(nba_ipsec.NbaIpsecError):
            ring.run(1)
        ring.close()


def test_ring_forms_switch_and_agree():
    """set_form switches a persistent ring between its two forms; both give the
    same bytes, lengths and counters as stream launches."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    p = gen.make_sas(1024, cfg_id=59)
    b = gen.make_batch(65536, "imix", 1024, cfg_id=59)
    da = [device.to_device(b, "cuda") for _ in range(2)]
    db_ = [device.to_device(b, "cuda") for _ in range(2)]
    with nba_ipsec.SATable(p, device=0, max_batch=b.n) as ta, \
            nba_ipsec.SATable(p, device=0, max_batch=b.n) as tb:
        ring = ta.ring([_slot(d) for d in da])
        assert ring.form == ring.PIPELINED
        ring.run(1)
        ring.set_form(ring.PERSISTENT)
        assert ring.form == ring.PERSISTENT
        ring.run(1)
        ring.set_form(ring.PIPELINED)
        ring.run(1)
        for _ in range(3):
            for d in db_:
                tb.process(*d.args(), n=b.n)
        torch.cuda.synchronize()
        for x, y in zip(da, db_):
            assert torch.equal(x.out_buf, y.out_buf) and torch.equal(x.out_len, y.out_len)
        assert np.array_equal(ta.sa_seq(), tb.sa_seq()) and ta.counters() == tb.counters()
        ring.close()


@pytest.mark.parametrize("form", ["pipelined", "persistent"])
def test_ring_sequence_overflow_matches_oracle(form):
    """SA counters near 2^32 - 1 (RFC 4303 §3.3.3: never cycle): the rings drop
    exactly the packets the oracle drops, over consecutive batches."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa, n = 32, 20000
    seq = np.full(n_sa, 0xFFFFFFFF - 700, np.uint32)
    seq[::3] = 0xFFFFFFFF
    seq[1::5] = 5
    p = gen.make_sas(n_sa, cfg_id=60)
    p = gen.SAParams(*[getattr(p, f) for f in ("spi", "tunnel_src", "tunnel_dst", "aes_key",
                                               "ctr_nonce", "hmac_key")], seq=seq)
    bs = [gen.make_batch(n, "imix", n_sa, cfg_id=60, batch=k) for k in range(2)]
    sas = oracle.make_sas(p)
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        ds = [device.to_device(b, "cuda") for b in bs]
        ring = t.ring([_slot(d) for d in ds])
        if form == "persistent":
            ring.set_form(ring.PERSISTENT)
        ring.run(2)
        torch.cuda.synchronize()
        for b in bs:
            oracle.process_batch(sas, n_sa, b, n_threads=8)
        ctr = oracle.Counters()
        for d, b in zip(ds, bs):
            o_out, o_len, _ = oracle.process_batch(sas, n_sa, b, n_threads=8, counters=ctr)
            g_out, g_len = device.fetch(d)
            assert np.array_equal(g_len, o_len)
            # only [0, out_len) of a slot is defined (a slot dropped in this round
            # still holds the previous round's packet)
            for i in np.nonzero(o_len)[0]:
                a, L = int(b.out_off[i]), int(o_len[i])
                assert np.array_equal(g_out[a:a + L], o_out[a:a + L])
        assert (g_len == 0).sum() > 0                          # drops happened
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa))
        ring.close()


@pytest.mark.parametrize("n", [1, 31, 100, 4737])
def test_pipelined_ring_small_batches(n):
    """Batches that leave most CTAs without packets (ppc = 32): the pipelined
    ring still equals the oracle over three rounds."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa = 8
    p = gen.make_sas(n_sa, cfg_id=61)
    bs = [gen.make_batch(n, "imix", n_sa, cfg_id=61, batch=k) for k in range(2)]
    sas = oracle.make_sas(p)
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        ds = [device.to_device(b, "cuda") for b in bs]
        ring = t.ring([_slot(d) for d in ds])
        assert ring.form == ring.PIPELINED
        ring.run(3)
        torch.cuda.synchronize()
        for _ in range(2):
            for b in bs:
                oracle.process_batch(sas, n_sa, b)
        for d, b in zip(ds, bs):
            o_out, o_len, _ = oracle.process_batch(sas, n_sa, b)
            g_out, g_len = device.fetch(d)
            assert np.array_equal(g_len, o_len) and np.array_equal(g_out, o_out)
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa))
        ring.close()


@pytest.mark.parametrize("graph", [False, True])
def test_run_batches_mid_rotation(graph, monkeypatch):
    """nba_ipsec_ring_run_batches stops mid-rotation and the next run continues
    from the cursor: 5 + 4 + 3 batches over 3 distinct slots (persistent and
    graph forms) equal the oracle over the same slot sequence."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    if graph:
        monkeypatch.setenv("NBA_IPSEC_RING_GRAPH", "1")
    n_sa, n = 61, 9000
    p = gen.make_sas(n_sa, cfg_id=57)
    hb = [gen.make_batch(n, s, n_sa, cfg_id=57, batch=i) for i, s in enumerate((64, "imix", 300))]
    sas = oracle.make_sas(p)
    ctr = oracle.Counters()
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        dbs = [device.to_device(b, "cuda") for b in hb]
        ring = t.ring([_slot(d) for d in dbs])
        assert ring.form == (nba_ipsec.Ring.GRAPH if graph else nba_ipsec.Ring.PIPELINED)
        last, k = {}, 0
        for nb in (5, 4, 3):
            ring.run_batches(nb)
            for _ in range(nb):
                o_out, o_len, _ = oracle.process_batch(sas, n_sa, hb[k % 3], n_threads=8, counters=ctr)
                last[k % 3] = (o_out, o_len.copy())
                k += 1
            assert ring.cursor == k % 3
        for s, (o_out, o_len) in last.items():
            g_out, g_len = device.fetch(dbs[s])
            assert np.array_equal(g_len, o_len)
            assert np.array_equal(g_out, o_out)
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa))
        assert t.counters() == ctr.as_dict()
        ring.close()


@pytest.mark.parametrize("n_sa,sizes", [(2500, (64, "imix")), (1024, (300, 300)), (1, (64, 1514))])
def test_pipelined_prologue_modes(n_sa, sizes):
    """The pipelined ring's prologue with the SA hash (n_sa > 1024), with
    per-SA counters indexed by the SA (one SA; 1024 SAs), one-length-bin
    batches (all packets one size: index order kept) and mixed ones; some
    invalid SAs and lengths; 4 runs of 2-3 batches against the oracle."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n = 30000
    p = gen.make_sas(n_sa, cfg_id=58)
    hb = [gen.make_batch(n, s, n_sa, cfg_id=58, batch=i) for i, s in enumerate(sizes)]
    hb[1].sa_idx[::101] = n_sa + 3
    hb[1].in_len[5::203] = 19
    sas = oracle.make_sas(p)
    ctr = oracle.Counters()
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        dbs = [device.to_device(b, "cuda") for b in hb]
        ring = t.ring([_slot(d) for d in dbs])
        if ring.form == nba_ipsec.Ring.ROLES:       # one-length slots: the role-split default
            ring.set_form(nba_ipsec.Ring.PIPELINED)
        assert ring.form == nba_ipsec.Ring.PIPELINED
        last, k = {}, 0
        for nb in (3, 2, 3, 2):
            ring.run_batches(nb)
            for _ in range(nb):
                o_out, o_len, _ = oracle.process_batch(sas, n_sa, hb[k % 2], n_threads=8, counters=ctr)
                last[k % 2] = (o_out, o_len.copy())
                k += 1
        for s, (o_out, o_len) in last.items():
            g_out, g_len = device.fetch(dbs[s])
            assert np.array_equal(g_len, o_len)
            assert np.array_equal(g_out, o_out)
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa))
        assert t.counters() == ctr.as_dict()
        ring.close()


@pytest.mark.parametrize("n_sa,sizes", [(16, [3000, 2500, 4000]), (1024, [20000, 20000, 9000]),
                                        (5000, [30000, 12000, 25000])])
def test_inbound_pipelined_ring_mixed_stream(n_sa, sizes, monkeypatch):
    """The software-pipelined inbound ring (k_in_fused_ring_pipe) on traffic
    with reordering, duplicates, stale replays, single-byte corruption,
    invalid SA indices and SPI mismatches: one rotation over the slots, then a
    partial rotation that replays the first two slots (every earlier packet
    now a replay), then seven batches in one launch, each run against the oracle's sequential receiver
    continuing from the same state: statuses, lengths, inner bytes, windows
    and counters."""
    import torch
    from harness import esp_source
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    monkeypatch.setenv("NBA_IPSEC_RING_IN_PIPE", "1")
    p = gen.make_sas(n_sa, cfg_id=70 + n_sa)
    b, out, ol = esp_source(p, sum(sizes), "imix", 70 + n_sa)
    r = gen.rng_for(6, salt=n_sa)
    bs, start = [], 0
    for k, n in enumerate(sizes):
        order = start + gen.arrival_order(n, n, r, reorder=9, dup=0.05, old=0.05, old_span=3000)
        order = np.clip(order, 0, sum(sizes) - 1)
        ib = gen.esp_batch(out, b.out_off, ol, b.sa_idx, order)
        kk = r.random(ib.n)
        ib.sa_idx[kk < 0.01] = n_sa + 7
        m = (kk >= 0.01) & (kk < 0.02)
        ib.sa_idx[m] = (ib.sa_idx[m] + 1) % n_sa
        for j in np.nonzero(r.random(ib.n) < 0.03)[0]:
            ib.in_buf[ib.in_off[j] + int(r.integers(0, ib.in_len[j]))] ^= np.uint8(r.integers(1, 256))
        bs.append(ib)
        start += n
    sas = oracle.make_sas(p)
    win = oracle.make_windows(sas, n_sa)
    ctr = oracle.InCounters()
    with nba_ipsec.SATable(p, device=0, max_batch=max(x.n for x in bs)) as t:
        t.enable_inbound()
        ds = [device.to_device(ib, "cuda", out_fill=0xA5) for ib in bs]
        sts = [torch.zeros(ib.n, dtype=torch.uint8, device="cuda") for ib in bs]
        ring = t.ring_inbound([(*d.args(), st, ib.n) for d, st, ib in zip(ds, sts, bs)])
        assert ring.form == ring.PIPELINED
        k = 0
        for nb in (len(bs), 2, 7):   # (7: every duplicate hash of the mod-3 rotation reused)
            ring.run_batches(nb)
            torch.cuda.synchronize()
            for _ in range(nb):
                ib = bs[k % len(bs)]
                o_out, o_len, o_st, _ = oracle.process_inbound(sas, win, n_sa, ib, counters=ctr)
                g_out, g_len = device.fetch(ds[k % len(bs)])
                assert np.array_equal(sts[k % len(bs)].cpu().numpy(), o_st), f"batch {k}: status"
                assert np.array_equal(g_len, o_len), f"batch {k}: out_len"
                for i in np.nonzero(o_len)[0]:
                    a, L = int(ib.out_off[i]), int(o_len[i])
                    assert np.array_equal(g_out[a:a + L], o_out[a:a + L]), f"batch {k}: packet {i}"
                k += 1
            top, bmp = t.replay_window()
            o_top, o_bmp = oracle.window_state(win, n_sa)
            assert np.array_equal(top, o_top) and np.array_equal(bmp, o_bmp)
            assert t.in_counters() == ctr.as_dict()
        ring.close()


@pytest.mark.parametrize("size,form", [(64, "pipelined"), (512, "pipelined"), (1024, "graph"),
                                       ("imix", "graph")])
def test_inbound_ring_form_choice(size, form):
    """Without overrides an inbound ring takes the pipelined form when every
    packet's outer length is <= 640 B and the graph form otherwise (DESIGN
    §5); either way the output equals the oracle's receiver."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa, n = 64, 3000
    p = gen.make_sas(n_sa, cfg_id=77)
    sas = oracle.make_sas(p)
    b = gen.make_batch(n, size, n_sa, cfg_id=77)
    e_out, e_len, _ = oracle.process_batch(sas, n_sa, b)
    ib = gen.esp_batch(e_out, b.out_off, e_len, b.sa_idx, np.arange(n))
    win = oracle.make_windows(oracle.make_sas(p), n_sa)
    o_out, o_len, o_st, _ = oracle.process_inbound(oracle.make_sas(p), win, n_sa, ib)
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        t.enable_inbound()
        d = device.to_device(ib, "cuda")
        st = torch.zeros(n, dtype=torch.uint8, device="cuda")
        ring = t.ring_inbound([(*d.args(), st, n)])
        assert ring.form == {"graph": ring.GRAPH, "pipelined": ring.PIPELINED}[form]
        ring.run_batches(1)
        torch.cuda.synchronize()
        g_out, g_len = device.fetch(d)
        assert np.array_equal(st.cpu().numpy(), o_st)
        assert np.array_equal(g_len, o_len)
        for i in np.nonzero(o_len)[0]:
            a, L = int(ib.out_off[i]), int(o_len[i])
            assert np.array_equal(g_out[a:a + L], o_out[a:a + L])
        ring.close()
