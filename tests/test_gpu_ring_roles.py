"""GPU parity of the role-split batch ring (nba_ipsec_ring form ROLES,
k_fused_ring_roles): sequencer CTAs assign every batch's sequence numbers
(RFC 4303 §3.3.3 as the oracle's steps 1-2: invalid SA or
length -> drop without consuming a number, a number that would pass 2^32 - 1
-> drop) and the other CTAs encrypt.  Against the oracle processing the same
batch sequence with carried SA state: whole output pools, out_len, final SA
counters, device counters -- over sequencer counts, SA counts (1 .. 2048),
batch sizes that leave most lane CTAs empty, one-slot rings (every batch
rewrites the same output slots), runs stopping mid-rotation, runs longer than
the record ring, invalid SAs / lengths and counters at 2^32 - 1."""
import numpy as np
import pytest

import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen

pytestmark = pytest.mark.gpu


def _slot(db):
    return (db.in_buf, db.in_off, db.in_len, db.sa_idx, db.out_buf, db.out_off, db.out_len, db.n)


def _roles_vs_oracle(p, n_sa, hb, runs, force=True, defined_only=False):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    sas = oracle.make_sas(p)
    ctr = oracle.Counters()
    R = len(hb)
    with nba_ipsec.SATable(p, device=0, max_batch=max(b.n for b in hb)) as t:
        dbs = [device.to_device(b, "cuda") for b in hb]
        ring = t.ring([_slot(d) for d in dbs])
        if force:
            ring.set_form(nba_ipsec.Ring.ROLES)
        assert ring.form == nba_ipsec.Ring.ROLES
        last, k = {}, 0
        for nb in runs:
            ring.run_batches(nb)
            for _ in range(nb):
                o_out, o_len, _ = oracle.process_batch(sas, n_sa, hb[k % R], n_threads=8, counters=ctr)
                last[k % R] = (o_out, o_len.copy())
                k += 1
            assert ring.cursor == k % R
        torch.cuda.synchronize()
        for s, (o_out, o_len) in last.items():
            g_out, g_len = device.fetch(dbs[s])
            assert np.array_equal(g_len, o_len), f"slot {s}: out_len differs"
            if defined_only:
                # only [0, out_len) of a packet's slot is defined: a packet dropped in
                # a later round leaves the earlier round's bytes there
                b = hb[s]
                for i in np.nonzero(o_len)[0]:
                    a, L = int(b.out_off[i]), int(o_len[i])
                    assert np.array_equal(g_out[a:a + L], o_out[a:a + L]), f"slot {s} packet {i}"
            elif not np.array_equal(g_out, o_out):
                d = np.nonzero(g_out != o_out)[0]
                raise AssertionError(f"slot {s}: {d.size} output bytes differ, first at {d[:8]}")
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa)), "final SA counters differ"
        assert t.counters() == ctr.as_dict()
        ring.close()


@pytest.mark.parametrize("npro", [1, 4, 9])
@pytest.mark.parametrize("n_sa,n,sizes", [(61, 9000, (64, "imix", 300)), (2048, 30000, (1514, 64)),
                                          (1, 20000, (64, 64))])
def test_roles_ring_matches_oracle(npro, n_sa, n, sizes, monkeypatch):
    """Sequencer counts 1 / 4 / 9, runs of 5 + 4 + 9 batches (past the record
    ring of 4), invalid SAs and lengths in slot 0."""
    if n > 16384 * npro:
        pytest.skip("a sequencer stashes at most 16,384 packets per batch")
    monkeypatch.setenv("NBA_IPSEC_ROLES_P", str(npro))
    p = gen.make_sas(n_sa, cfg_id=71)
    hb = [gen.make_batch(n, s, n_sa, cfg_id=71, batch=i) for i, s in enumerate(sizes)]
    hb[0].sa_idx[::97] = n_sa + 1
    hb[0].in_len[3::211] = 19
    hb[0].in_len[7::223] = 1501
    _roles_vs_oracle(p, n_sa, hb, [5, 4, 9])


def test_roles_ring_one_slot(monkeypatch):
    """One slot: every batch rewrites the same output slots with new sequence
    numbers; the last batch's bytes must be what stays."""
    p = gen.make_sas(16, cfg_id=72)
    hb = [gen.make_batch(40000, 64, 16, cfg_id=72)]
    _roles_vs_oracle(p, 16, hb, [7, 1, 6], force=False)     # one length: the default form


@pytest.mark.parametrize("n", [1, 31, 100, 4737, 65536])
def test_roles_ring_batch_sizes(n):
    """Batches that leave most lane CTAs (and sequencer ranges) empty, up to
    the bench's 65,536 packets."""
    p = gen.make_sas(8, cfg_id=73)
    hb = [gen.make_batch(n, s, 8, cfg_id=73, batch=k) for k, s in enumerate(("imix", 64))]
    _roles_vs_oracle(p, 8, hb, [3, 2])


def test_roles_ring_sequence_overflow():
    """SA counters near 2^32 - 1 over consecutive batches: the sequencers drop
    exactly the packets the oracle drops (and no later packet of that SA)."""
    n_sa, n = 32, 20000
    seq = np.full(n_sa, 0xFFFFFFFF - 700, np.uint32)
    seq[::3] = 0xFFFFFFFF
    seq[1::5] = 5
    p = gen.make_sas(n_sa, cfg_id=74)
    p = gen.SAParams(*[getattr(p, f) for f in ("spi", "tunnel_src", "tunnel_dst", "aes_key",
                                               "ctr_nonce", "hmac_key")], seq=seq)
    hb = [gen.make_batch(n, "imix", n_sa, cfg_id=74, batch=k) for k in range(2)]
    _roles_vs_oracle(p, n_sa, hb, [2, 3], defined_only=True)


def test_roles_ring_then_other_paths():
    """A role-split run, then process_batch and a pipelined run on the same
    table continue the SA counters exactly (the device state it leaves)."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa, n = 100, 25000
    p = gen.make_sas(n_sa, cfg_id=75)
    hb = [gen.make_batch(n, 64, n_sa, cfg_id=75, batch=k) for k in range(2)]
    sas = oracle.make_sas(p)
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        dbs = [device.to_device(b, "cuda") for b in hb]
        ring = t.ring([_slot(d) for d in dbs])
        assert ring.form == nba_ipsec.Ring.ROLES
        ring.run_batches(5)                    # slots 0 1 0 1 0
        for k in range(5):
            oracle.process_batch(sas, n_sa, hb[k % 2])
        t.process(*dbs[1].args(), n=n)         # slot 1 through process_batch
        o1 = oracle.process_batch(sas, n_sa, hb[1])
        ring.set_form(nba_ipsec.Ring.PIPELINED)
        ring.run_batches(1)                    # cursor 1: slot 1 again
        o1 = oracle.process_batch(sas, n_sa, hb[1])
        ring.set_form(nba_ipsec.Ring.ROLES)
        ring.run_batches(2)                    # slots 0, 1
        o0 = oracle.process_batch(sas, n_sa, hb[0])
        o1 = oracle.process_batch(sas, n_sa, hb[1])
        torch.cuda.synchronize()
        for d, (o_out, o_len, _) in zip(dbs, (o0, o1)):
            g_out, g_len = device.fetch(d)
            assert np.array_equal(g_len, o_len) and np.array_equal(g_out, o_out)
        assert np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa))
        ring.close()


@pytest.mark.parametrize("npro,n_sa,n", [(4, 61, 9000), (6, 1024, 65536), (2, 2048, 30000), (5, 7, 100)])
def test_roles_ring_sorted_mode(npro, n_sa, n, monkeypatch):
    """Sorted mode (mixed-length rings with more slots than the record ring):
    per batch the sequencers sort each lane CTA's packets by length and place
    runs of 32 on the lane warps by cumulative cost, so a packet slot changes
    lanes between uses of a ring slot -- 6 slots of mixed traffic (IMIX, 64 B,
    1514 B), invalid SAs / lengths, runs of 7 + 5 + 13 batches."""
    monkeypatch.setenv("NBA_IPSEC_ROLES_P", str(npro))
    p = gen.make_sas(n_sa, cfg_id=76)
    sizes = ("imix", 64, "imix", 1514, "imix", 300)
    hb = [gen.make_batch(n, s, n_sa, cfg_id=76, batch=i) for i, s in enumerate(sizes)]
    hb[0].sa_idx[::89] = n_sa + 2
    hb[2].in_len[4::97] = 19
    _roles_vs_oracle(p, n_sa, hb, [7, 5, 13])


def test_roles_ring_sorted_mode_overflow():
    """Sorted mode with SA counters at / near 2^32 - 1 over 6 slots."""
    n_sa, n = 32, 20000
    seq = np.full(n_sa, 0xFFFFFFFF - 1500, np.uint32)
    seq[::3] = 0xFFFFFFFF
    p = gen.make_sas(n_sa, cfg_id=77)
    p = gen.SAParams(*[getattr(p, f) for f in ("spi", "tunnel_src", "tunnel_dst", "aes_key",
                                               "ctr_nonce", "hmac_key")], seq=seq)
    hb = [gen.make_batch(n, "imix", n_sa, cfg_id=77, batch=k) for k in range(6)]
    _roles_vs_oracle(p, n_sa, hb, [6, 5], defined_only=True)


@pytest.mark.parametrize("sorted_mode", [False, True])
def test_roles_ring_sequencer_plain_loads(sorted_mode, monkeypatch):
    """The sequencers' fallback without bulk staging (SA index / length arrays
    not 16-byte aligned take it; forced here), fixed and sorted lane slots."""
    monkeypatch.setenv("NBA_IPSEC_ROLES_NOSTAGE", "1")
    p = gen.make_sas(40, cfg_id=78)
    sizes = ("imix", 64, "imix", 1514, 300) if sorted_mode else (64, 64)
    hb = [gen.make_batch(7001, s, 40, cfg_id=78, batch=i) for i, s in enumerate(sizes)]
    hb[0].sa_idx[::61] = 77
    _roles_vs_oracle(p, 40, hb, [6, 7])


@pytest.mark.parametrize("sizes", [(64, 64, 64), ("imix", 300)])
def test_roles_ring_without_bootstrap(sizes, monkeypatch):
    """Fixed-slot rings with the sequencers numbering batch 0 too
    (NBA_IPSEC_ROLES_NOBOOT; by default every CTA numbers a launch's first
    batch), runs of 4 + 1 + 6 batches."""
    monkeypatch.setenv("NBA_IPSEC_ROLES_NOBOOT", "1")
    p = gen.make_sas(200, cfg_id=79)
    hb = [gen.make_batch(12000, s, 200, cfg_id=79, batch=i) for i, s in enumerate(sizes)]
    hb[0].sa_idx[::71] = 999
    _roles_vs_oracle(p, 200, hb, [4, 1, 6])


def test_roles_form_refused_where_it_does_not_fit():
    """set_form(ROLES) is refused (NBA_IPSEC_EINVAL) for slots it does not fit:
    more than 2048 SAs, or more than 512 packets per encrypting CTA; the ring
    keeps its form and still equals the oracle."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    for n_sa, n in ((2500, 5000), (16, 100_000)):
        p = gen.make_sas(n_sa, cfg_id=80)
        b = gen.make_batch(n, 64, n_sa, cfg_id=80)
        sas = oracle.make_sas(p)
        with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
            d = device.to_device(b, "cuda")
            ring = t.ring([_slot(d)])
            form = ring.form
            assert form != nba_ipsec.Ring.ROLES
            with pytest.raises(nba_ipsec.NbaIpsecError):
                ring.set_form(nba_ipsec.Ring.ROLES)
            assert ring.form == form
            ring.run_batches(2)
            torch.cuda.synchronize()
            oracle.process_batch(sas, n_sa, b)
            o_out, o_len, _ = oracle.process_batch(sas, n_sa, b)
            g_out, g_len = device.fetch(d)
            assert np.array_equal(g_len, o_len) and np.array_equal(g_out, o_out)
            ring.close()


@pytest.mark.parametrize("sizes", [(64,), (64, "imix")])
def test_roles_ring_many_slots(sizes):
    """More slots than the lanes' shared-memory slot table holds (179): the
    lanes read the slot arguments from global memory; 190 small slots,
    fixed-slot (one length) and sorted (mixed) modes, 250 + 140 batches."""
    n_sa, n, R = 24, 300, 190
    p = gen.make_sas(n_sa, cfg_id=81)
    hb = [gen.make_batch(n, sizes[k % len(sizes)], n_sa, cfg_id=81, batch=k) for k in range(R)]
    _roles_vs_oracle(p, n_sa, hb, [250, 140], force=False)


def test_roles_ring_slots_of_different_sizes():
    """Slots of 65,536 / 1,000 / 30,000 / 7 packets in one ring (the lanes'
    packet -> lane mapping changes from slot to slot, the bootstrap takes the
    first batch's), 9 + 6 batches."""
    n_sa = 300
    p = gen.make_sas(n_sa, cfg_id=82)
    hb = [gen.make_batch(n, 64, n_sa, cfg_id=82, batch=k) for k, n in enumerate((65536, 1000, 30000, 7))]
    _roles_vs_oracle(p, n_sa, hb, [9, 6], force=False)
