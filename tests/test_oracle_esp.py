"""Pins for the oracle's ESP composition (tiers T2-T4): the worked example,
an independent pyca+hmac composition, decap round trips, invariants and edge
cases.  None of these values come from the CUDA path."""
import struct

import numpy as np
import pytest

import oracle
import pyca_esp
from golden import load
from paper_conf_eurosys_kimjlmsm15_b200 import gen

EX = load("esp_worked_example.txt")


def _example_sa():
    r = EX["sa"]
    p = gen.SAParams(
        spi=np.array([int(r["spi"], 16)], np.uint32),
        tunnel_src=np.array([int(r["tunnel_src"], 16)], np.uint32),
        tunnel_dst=np.array([int(r["tunnel_dst"], 16)], np.uint32),
        aes_key=np.frombuffer(bytes.fromhex(r["aes_key"]), np.uint8)[None, :].copy(),
        ctr_nonce=np.frombuffer(bytes.fromhex(r["nonce"]), np.uint8)[None, :].copy(),
        hmac_key=np.frombuffer(bytes.fromhex(r["hmac_key"]), np.uint8)[None, :].copy(),
        seq=np.array([int(r["seq0"], 16)], np.uint32))
    return p


def _batch_from_packets(pkts, sa_idx, stride=2048, off=142):
    n = len(pkts)
    buf = np.zeros(max(n, 1) * stride, np.uint8)
    in_off = np.array([stride * i + off for i in range(n)], np.uint32)
    for i, p in enumerate(pkts):
        buf[in_off[i]:in_off[i] + len(p)] = np.frombuffer(bytes(p), np.uint8)
    return gen.Batch(n=n, in_buf=buf, in_off=in_off,
                     in_len=np.array([len(p) for p in pkts], np.uint16),
                     sa_idx=np.asarray(sa_idx, np.uint32), out_off=in_off.copy(),
                     out_pool_bytes=max(n, 1) * stride,
                     frame_len=np.array([len(p) + 14 for p in pkts], np.uint32))


def _slot(out_buf, b, i, L):
    return out_buf[b.out_off[i]:b.out_off[i] + L].tobytes()


def test_worked_example_byte_exact():
    """two packets on one SA, seq 1 and 2, pad 0 and 3."""
    p = _example_sa()
    sas = oracle.make_sas(p)
    pk = [bytes.fromhex(EX["pkt1"]["inner"]), bytes.fromhex(EX["pkt2"]["inner"])]
    b = _batch_from_packets(pk, [0, 0])
    out, out_len, ctr = oracle.process_batch(sas, 1, b)
    for i, name in enumerate(["pkt1", "pkt2"]):
        exp = bytes.fromhex(EX[name]["output"])
        assert int(out_len[i]) == len(exp)
        assert _slot(out, b, i, len(exp)) == exp
    assert oracle.sa_seq(sas, 1).tolist() == [2]
    assert ctr.as_dict() == dict(pkts_ok=2, pkts_dropped=0, bytes_in=73, bytes_out=176, batches=1)


def test_worked_example_intermediates():
    """Intermediate values of the example pin each step separately."""
    r = EX["sa"]
    key, nonce = bytes.fromhex(r["aes_key"]), bytes.fromhex(r["nonce"])
    e1 = EX["pkt1"]
    assert oracle.aes128_encrypt(key, bytes.fromhex(e1["ctrblk1"])).hex() == e1["ks0"]
    icb = bytes.fromhex(e1["ctrblk1"])
    assert oracle.ctr_xcrypt(key, icb, bytes.fromhex(e1["T"])).hex() == e1["E"]
    mac = oracle.hmac_sha1(bytes.fromhex(r["hmac_key"]), bytes.fromhex(e1["H"] + e1["E"]))
    assert mac.hex() == e1["hmac_full"]
    assert oracle.ipv4_checksum(bytes.fromhex(e1["outer"])) == 0


def _random_sas(n_sa, seed):
    return gen.make_sas(n_sa, cfg_id=100 + seed)


def test_vs_independent_pyca_composition():
    """Third composition (pyca AES-CTR + stdlib hmac) on random packets D∈[20,1500]."""
    rng = np.random.default_rng(11)
    n, n_sa = 400, 7
    p = _random_sas(n_sa, 1)
    D = rng.integers(20, 1501, n)
    b = gen.make_batch(n, 64, n_sa, cfg_id=101, in_len_override=D)
    sas = oracle.make_sas(p)
    out, out_len, ctr = oracle.process_batch(sas, n_sa, b)
    seq = p.seq.astype(np.int64).copy()
    for i in range(n):
        s = int(b.sa_idx[i])
        seq[s] += 1
        P = b.in_buf[b.in_off[i]:b.in_off[i] + int(b.in_len[i])].tobytes()
        exp = pyca_esp.encap(int(p.spi[s]), p.aes_key[s], p.ctr_nonce[s], p.hmac_key[s],
                             int(p.tunnel_src[s]), int(p.tunnel_dst[s]), int(seq[s]), P)
        assert int(out_len[i]) == len(exp)
        assert _slot(out, b, i, len(exp)) == exp, i
    assert oracle.sa_seq(sas, n_sa).tolist() == seq.tolist()


def test_invariants_and_round_trip():
    """T3: decap recovers P (oracle and pyca), lengths, pad, seq/IV, checksum, ICV."""
    n, n_sa = 300, 5
    p = _random_sas(n_sa, 2)
    rng = np.random.default_rng(12)
    D = rng.integers(20, 1501, n)
    b = gen.make_batch(n, 64, n_sa, cfg_id=102, in_len_override=D)
    sas = oracle.make_sas(p)
    out, out_len, _ = oracle.process_batch(sas, n_sa, b)
    last = {}
    for i in range(n):
        s = int(b.sa_idx[i])
        Dv = int(b.in_len[i])
        L = int(out_len[i])
        pad = (-(Dv + 2)) % 4
        C = Dv + pad + 2
        assert L == 48 + C == Dv + pad + 50 and C % 4 == 0
        pkt = _slot(out, b, i, L)
        P = b.in_buf[b.in_off[i]:b.in_off[i] + Dv].tobytes()
        assert oracle.ipv4_checksum(pkt[:20]) == 0                       # folds to 0xFFFF
        assert struct.unpack("!H", pkt[2:4])[0] == L and pkt[1] == P[1]
        assert pkt[6:10] == b"\x40\x00\x40\x32"
        spi, q = struct.unpack("!II", pkt[20:28])
        assert spi == int(p.spi[s]) and pkt[28:36] == struct.pack("!Q", q)  # IV = BE64(seq)
        assert q == last.get(s, 0) + 1                                    # contiguous per SA
        last[s] = q
        rc, inner, q2 = oracle.decap(sas, s, pkt)
        assert rc == 0 and inner == P and q2 == q
        inner2, q3 = pyca_esp.decap(p.aes_key[s], p.ctr_nonce[s], p.hmac_key[s], pkt)
        assert inner2 == P and q3 == q
        if i < 40:   # any single bit flip in H||E||ICV fails authentication
            j = 24 + int(rng.integers(0, L - 24))       # seq..ICV (an SPI flip is EFORMAT)
            bad = bytearray(pkt)
            bad[j] ^= 1 << int(rng.integers(0, 8))
            assert oracle.decap(sas, s, bytes(bad))[0] == -3


@pytest.mark.parametrize("D,pad", [(20, 2), (21, 1), (22, 0), (23, 3), (1497, 1), (1498, 0),
                                   (1499, 3), (1500, 2)])
def test_edge_lengths_padding(D, pad):
    p = _random_sas(1, 3)
    b = gen.make_batch(1, 64, 1, cfg_id=103, in_len_override=[D])
    sas = oracle.make_sas(p)
    out, out_len, ctr = oracle.process_batch(sas, 1, b)
    assert int(out_len[0]) == 48 + D + pad + 2
    rc, inner, _ = oracle.decap(sas, 0, _slot(out, b, 0, int(out_len[0])))
    assert rc == 0 and len(inner) == D


def test_drops_consume_no_seq():
    """T4: invalid lengths and SA indices drop without consuming a sequence number."""
    p = _random_sas(2, 4)
    D = [50, 0, 19, 1501, 50, 50, 60]
    sa = [0, 0, 0, 0, 2, 1, 0]          # sa_idx 2 >= n_sa
    b = gen.make_batch(7, 64, 2, cfg_id=104, in_len_override=D, sa_idx_override=sa)
    sas = oracle.make_sas(p)
    out, out_len, ctr = oracle.process_batch(sas, 2, b)
    assert out_len.tolist() == [100, 0, 0, 0, 0, 100, 112]
    assert oracle.sa_seq(sas, 2).tolist() == [2, 1]
    assert struct.unpack("!I", _slot(out, b, 6, 112)[24:28])[0] == 2
    assert ctr.as_dict() == dict(pkts_ok=3, pkts_dropped=4, bytes_in=160, bytes_out=312,
                                 batches=1)


def test_seq_overflow_drops_and_counter_stops():
    """RFC 4303 §3.3.3: the 32-bit counter must not cycle; packets past 2^32-1 drop."""
    p = _random_sas(2, 5)
    p.seq[:] = [0xFFFFFFFD, 7]
    sa = [0, 1, 0, 0, 0, 1]
    b = gen.make_batch(6, 64, 2, cfg_id=105, sa_idx_override=sa)
    sas = oracle.make_sas(p)
    out, out_len, ctr = oracle.process_batch(sas, 2, b)
    assert out_len.tolist() == [100, 100, 100, 0, 0, 100]
    assert oracle.sa_seq(sas, 2).tolist() == [0xFFFFFFFF, 9]
    q = struct.unpack("!I", _slot(out, b, 2, 100)[24:28])[0]
    assert q == 0xFFFFFFFF
    # a fully exhausted SA drops everything
    out, out_len, ctr = oracle.process_batch(sas, 2, b)
    assert out_len.tolist() == [0, 100, 0, 0, 0, 100]


def test_empty_and_single_batches():
    p = _random_sas(1, 6)
    sas = oracle.make_sas(p)
    b0 = gen.make_batch(0, 64, 1, cfg_id=106)
    _, ol, ctr = oracle.process_batch(sas, 1, b0)
    assert ol.size == 0 and ctr.as_dict()["batches"] == 0
    b1 = gen.make_batch(1, 1514, 1, cfg_id=106)
    _, ol, ctr = oracle.process_batch(sas, 1, b1)
    assert ol.tolist() == [1552]


def test_threaded_oracle_identical_to_sequential():
    """SA-partitioned threads (s mod T) give byte-identical results."""
    n, n_sa = 2000, 33
    p = _random_sas(n_sa, 7)
    b = gen.make_batch(n, "imix", n_sa, cfg_id=107)
    b.in_len[::97] = 5            # some drops
    s1, s4 = oracle.make_sas(p), oracle.make_sas(p)
    o1, l1, c1 = oracle.process_batch(s1, n_sa, b, n_threads=1)
    o4, l4, c4 = oracle.process_batch(s4, n_sa, b, n_threads=4)
    assert np.array_equal(o1, o4) and np.array_equal(l1, l4)
    assert c1.as_dict() == c4.as_dict()
    assert np.array_equal(oracle.sa_seq(s1, n_sa), oracle.sa_seq(s4, n_sa))


def test_generator_shapes():
    b = gen.make_batch(12, "imix", 4, cfg_id=4)
    assert set(b.frame_len.tolist()) <= {64, 594, 1514}
    assert (b.in_off % 16 == 14).all()
    big = gen.make_batch(65536, "imix", 1024, cfg_id=4)
    assert np.bincount(np.searchsorted([64, 594, 1514], big.frame_len)).tolist() == \
        [38229, 21845, 5462]
