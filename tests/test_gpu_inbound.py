"""GPU parity for ESP inbound: the CUDA path (k_in_fused ->
k_in_replay -> k_in_decide, through the C ABI) against the sequential oracle,
packet by packet: status, out_len, the inner bytes [0, out_len), the final
receive windows (right edge and bitmap) and the device counters.  Inputs are
ESP packets made by the OUTBOUND ORACLE from seeded gen batches, rearranged
(reordering, replays, stale packets, corruption, bad SA indices) by gen."""
import numpy as np
import pytest

from harness import assert_same_inbound, esp_source, gpu_inbound_run, oracle_inbound_run
from paper_conf_eurosys_kimjlmsm15_b200 import gen

pytestmark = pytest.mark.gpu


def _batches(b, out, ol, sizes, seed, **mix):
    r = gen.rng_for(seed, salt=11)
    bs, start = [], 0
    for n in sizes:
        order = (gen.arrival_order(b.n, n, r, **mix) + start) % b.n
        bs.append(gen.esp_batch(out, b.out_off, ol, b.sa_idx, order))
        start += n
    return bs


@pytest.mark.parametrize("cfg", [2, 3, 4])
def test_full_size_round_trip(cfg):
    """BASELINE configs[1..3] traffic (65,536 packets, 1024 SAs) decapsulated in
    order: every packet accepted and equal to the original inner datagram."""
    c = gen.CONFIGS[cfg]
    p = gen.make_sas(c["n_sa"], cfg_id=cfg)
    b, out, ol = esp_source(p, c["n"], c["size"], cfg)
    ib = gen.esp_batch(out, b.out_off, ol, b.sa_idx, np.arange(b.n))
    g = gpu_inbound_run(p, [ib])
    assert_same_inbound(g, oracle_inbound_run(p, [ib]), [ib])
    go, gl, gs = g[0][0]
    assert (gs == 0).all()
    for i in range(0, b.n, 997):
        D = int(b.in_len[i])
        assert int(gl[i]) == D
        assert go[ib.out_off[i]:ib.out_off[i] + D].tobytes() == \
            b.in_buf[b.in_off[i]:b.in_off[i] + D].tobytes()


@pytest.mark.parametrize("n_sa,sizes", [(16, [3000, 2500, 4000]), (3, [1200, 1200]),
                                        (1024, [20000, 20000])])
def test_mixed_stream(n_sa, sizes):
    """Reordering, duplicates, stale replays, corruption, invalid SA indices and
    SPI mismatches over consecutive batches (the window carries over)."""
    p = gen.make_sas(n_sa, cfg_id=90 + n_sa)
    b, out, ol = esp_source(p, sum(sizes), "imix", 90 + n_sa)
    bs = _batches(b, out, ol, sizes, 90 + n_sa, reorder=9, dup=0.05, old=0.05, old_span=3000)
    r = gen.rng_for(5, salt=n_sa)
    for ib in bs:
        k = r.random(ib.n)
        ib.sa_idx[k < 0.01] = n_sa + 7
        m = (k >= 0.01) & (k < 0.02)
        ib.sa_idx[m] = (ib.sa_idx[m] + 1) % n_sa
        hit = np.nonzero(r.random(ib.n) < 0.03)[0]
        for j in hit:
            ib.in_buf[ib.in_off[j] + int(r.integers(0, ib.in_len[j]))] ^= np.uint8(r.integers(1, 256))
    g = gpu_inbound_run(p, bs)
    o = oracle_inbound_run(p, bs)
    assert_same_inbound(g, o, bs)
    kinds = np.bincount(np.concatenate([x[2] for x in o[0]]), minlength=6)
    assert kinds[0] and kinds[2] and kinds[3] and kinds[4]


def test_same_batch_twice_and_single_sa_duplicates():
    """All packets on one SA with many copies of the same numbers (hash keys
    repeated), then the whole batch replayed: everything is a replay."""
    p = gen.make_sas(1, cfg_id=93)
    b, out, ol = esp_source(p, 700, 64, 93)
    r = gen.rng_for(93, salt=3)
    order = np.sort(r.integers(0, 700, 3000))
    ib = gen.esp_batch(out, b.out_off, ol, b.sa_idx, order)
    ib2 = gen.esp_batch(out, b.out_off, ol, b.sa_idx, order)
    g = gpu_inbound_run(p, [ib, ib2])
    o = oracle_inbound_run(p, [ib, ib2])
    assert_same_inbound(g, o, [ib, ib2])
    assert (o[0][1][2] == 3).all()


def test_resumed_window_and_ragged_sizes():
    """SAs created with seq > 0 (reading B6) and batch sizes that leave ragged
    tiles / lane groups; a 1-packet batch."""
    n_sa = 8
    p = gen.make_sas(n_sa, cfg_id=94)
    b, out, ol = esp_source(p, 4000, "imix", 94)
    q = p.copy()
    q.seq[:] = np.array([0, 5, 40, 100, 1, 0, 63, 64], np.uint32)
    r = gen.rng_for(94, salt=1)
    bs = []
    start = 0
    for n in (1, 31, 257, 1000, 2711):
        order = (gen.arrival_order(b.n, n, r, reorder=5, dup=0.02) + start) % b.n
        bs.append(gen.esp_batch(out, b.out_off, ol, b.sa_idx, order))
        start += n
    assert_same_inbound(gpu_inbound_run(q, bs), oracle_inbound_run(q, bs), bs)


def test_packed_unaligned_layout():
    """Back-to-back packets at arbitrary alignment (layout="packed")."""
    n_sa = 32
    p = gen.make_sas(n_sa, cfg_id=95)
    b, out, ol = esp_source(p, 3000, "imix", 95)
    r = gen.rng_for(95, salt=2)
    order = gen.arrival_order(b.n, 3000, r, reorder=4, dup=0.03)
    ib = gen.esp_batch(out, b.out_off, ol, b.sa_idx, order, layout="packed")
    assert_same_inbound(gpu_inbound_run(p, [ib]), oracle_inbound_run(p, [ib]), [ib])


def test_empty_batch_and_errors():
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    p = gen.make_sas(4, cfg_id=96)
    t = nba_ipsec.SATable(p, max_batch=64)
    z = torch.zeros(1, dtype=torch.int32, device="cuda")
    with pytest.raises(nba_ipsec.NbaIpsecError):      # not enabled yet
        t.process_inbound(z, z, z, z, z, z, z, n=1)
    t.enable_inbound()
    t.process_inbound(z, z, z, z, z, z, z, n=0)       # no-op
    with pytest.raises(nba_ipsec.NbaIpsecError):
        t.process_inbound(z, z, z, z, z, z, z, n=65)
    top, bmp = t.replay_window()
    assert top.tolist() == [0] * 4 and bmp.tolist() == [0] * 4
    assert t.in_counters()["batches"] == 0
    t.close()


def test_last_cta_scan_fallback(monkeypatch):
    """k_in_replay's per-SA row scans on the last CTA (no grid barrier)."""
    monkeypatch.setenv("NBA_IPSEC_NO_GRIDSYNC", "1")
    n_sa = 40
    p = gen.make_sas(n_sa, cfg_id=97)
    b, out, ol = esp_source(p, 9000, "imix", 97)
    bs = _batches(b, out, ol, [4000, 5000], 97, reorder=7, dup=0.05, old=0.04, old_span=2000)
    assert_same_inbound(gpu_inbound_run(p, bs), oracle_inbound_run(p, bs), bs)


def test_reset_inbound_replays_same_traffic():
    """nba_ipsec_reset_inbound restores the initial windows: the same batch is
    accepted again with identical output (the bench's steady-state protocol)."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa = 64
    p = gen.make_sas(n_sa, cfg_id=98)
    b, out, ol = esp_source(p, 5000, "imix", 98)
    ib = gen.esp_batch(out, b.out_off, ol, b.sa_idx, np.arange(b.n))
    t = nba_ipsec.SATable(p, max_batch=b.n)
    t.enable_inbound()
    db = device.to_device(ib, "cuda")
    t.process_inbound(*db.args(), n=ib.n)
    o1, l1 = device.fetch(db)
    w1 = t.replay_window()
    t.process_inbound(*db.args(), n=ib.n)          # all replays now
    _, l2 = device.fetch(db)
    assert (l2 == 0).all()
    t.reset_inbound()
    db.out_buf.zero_()
    t.process_inbound(*db.args(), n=ib.n)
    o3, l3 = device.fetch(db)
    assert np.array_equal(l1, l3) and (l1 > 0).all()
    assert np.array_equal(o1, o3)
    w3 = t.replay_window()
    assert np.array_equal(w1[0], w3[0]) and np.array_equal(w1[1], w3[1])
    c = t.in_counters()
    assert c["pkts_ok"] == 2 * ib.n and c["drop_replay"] == ib.n and c["batches"] == 3
    t.close()
    torch.cuda.synchronize()


def test_long_padding_and_bad_trailers():
    """RFC 4303 §2.4 padding of up to 255 bytes (the kernel checks pad bytes
    beyond its last two words by reading back its own output), wrong pad
    bytes at every distance from the end, wrong next header, D < 20, and a
    non-counter IV -- built with the independent pyca composition."""
    import pyca_esp
    from test_oracle_inbound import _packets_batch
    p = gen.make_sas(1, cfg_id=99)
    kw = dict(spi=int(p.spi[0]), key=p.aes_key[0], nonce=p.ctr_nonce[0], hkey=p.hmac_key[0],
              src=int(p.tunnel_src[0]), dst=int(p.tunnel_dst[0]))
    r = np.random.default_rng(99)
    pk, q = [], 0
    for plen in (0, 1, 2, 3, 5, 6, 7, 8, 13, 14, 15, 16, 17, 63, 64, 100, 200, 254, 255):
        for bad in (None, "pad", "nh"):
            D = int(r.integers(20, 300))
            D -= (D + plen + 2) % 4                       # C = 0 mod 4
            if D < 20:
                D += 4
            P = bytes([0x45, 0]) + bytes(r.integers(0, 256, D - 2, dtype=np.uint8))
            pad = bytearray(range(1, plen + 1))
            nh = 4
            if bad == "pad" and plen:
                pad[int(r.integers(0, plen))] ^= 0x40
            if bad == "nh":
                nh = 41
            q += 1
            T = P + bytes(pad) + bytes([plen, nh])
            iv = bytes(r.integers(0, 256, 8, dtype=np.uint8)) if q % 3 == 0 else None
            pk.append(pyca_esp.encap_raw(kw["spi"], kw["key"], kw["nonce"], kw["hkey"], kw["src"],
                                         kw["dst"], q, T=T, iv=iv))
    # D < 20 once the long padding is stripped
    pk.append(pyca_esp.encap_raw(kw["spi"], kw["key"], kw["nonce"], kw["hkey"], kw["src"], kw["dst"],
                                 q + 1, T=bytes([0x45, 0]) + bytes(14) + bytes(range(1, 7)) + bytes([6, 4])))
    ib = _packets_batch([x for x in pk if len(x) <= 1552], [0] * len([x for x in pk if len(x) <= 1552]))
    g = gpu_inbound_run(p, [ib])
    o = oracle_inbound_run(p, [ib])
    assert_same_inbound(g, o, [ib])
    st = o[0][0][2]
    assert (st == 0).sum() >= 15 and (st == 5).sum() >= 30
