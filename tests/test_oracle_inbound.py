"""Pins for the oracle's ESP inbound path (readings B1..B9 in
DESIGN.md): round trips through the (already pinned) outbound oracle, an
independent Python composition (pyca AES-CTR + stdlib hmac + a set-based
receive window), hand-derived RFC 4303 §3.4.3 window sequences, and the status
class of every single-byte corruption.  None of these values come from the
CUDA path."""
import struct

import numpy as np

import oracle
import pyca_esp
from paper_conf_eurosys_kimjlmsm15_b200 import gen

OK, DSA, DFMT, DREP, DAUTH, DTRL = range(6)


def _outbound(params, n, size, cfg_id, batch=0):
    b = gen.make_batch(n, size, len(params.spi), cfg_id=cfg_id, batch=batch)
    sas = oracle.make_sas(params)
    out, ol, _ = oracle.process_batch(sas, len(params.spi), b)
    return b, out, ol


def _packets_batch(pkts, sa_idx):
    n = len(pkts)
    lens = np.array([len(p) for p in pkts], np.int64)
    off = np.concatenate([[0], np.cumsum(lens)[:-1]]).astype(np.int64) if n else np.zeros(0)
    buf = np.zeros(int(lens.sum()) + 16, np.uint8)
    for i, p in enumerate(pkts):
        buf[off[i]:off[i] + len(p)] = np.frombuffer(bytes(p), np.uint8)
    return gen.esp_batch(buf, off, lens, np.asarray(sa_idx), np.arange(n))


def _run(params, b, win=None):
    sas = oracle.make_sas(params)
    n_sa = len(params.spi)
    win = win if win is not None else oracle.make_windows(sas, n_sa)
    out, ol, st, ctr = oracle.process_inbound(sas, win, n_sa, b)
    return out, ol, st, ctr, win


def _one_sa(seq0=0):
    p = gen.make_sas(1, cfg_id=71)
    p.seq[:] = seq0
    return p


def _pk(p, q, P=None, **kw):
    P = P if P is not None else bytes([0x45, 0]) + bytes(range(2, 50))
    return pyca_esp.encap(int(p.spi[0]), p.aes_key[0], p.ctr_nonce[0], p.hmac_key[0],
                          int(p.tunnel_src[0]), int(p.tunnel_dst[0]), q, P) if not kw else \
        pyca_esp.encap_raw(int(p.spi[0]), p.aes_key[0], p.ctr_nonce[0], p.hmac_key[0],
                           int(p.tunnel_src[0]), int(p.tunnel_dst[0]), q, **kw)


def test_round_trip_identity():
    """outbound oracle -> inbound oracle returns every inner datagram; the
    window ends at the outbound counter with all recent numbers marked."""
    params = gen.make_sas(16, cfg_id=61)
    b, out, ol = _outbound(params, 700, "imix", 61)
    assert (ol > 0).all()
    ib = gen.esp_batch(out, b.out_off, ol, b.sa_idx, np.arange(b.n))
    o2, l2, st, ctr, win = _run(params, ib)
    assert (st == OK).all()
    for i in range(b.n):
        D = int(b.in_len[i])
        assert int(l2[i]) == D
        assert o2[ib.out_off[i]:ib.out_off[i] + D].tobytes() == \
            b.in_buf[b.in_off[i]:b.in_off[i] + D].tobytes()
    top, bmp = oracle.window_state(win, 16)
    cnt = np.bincount(b.sa_idx, minlength=16)
    assert top.tolist() == cnt.tolist()
    for s in range(16):
        c = int(cnt[s])
        assert int(bmp[s]) == ((1 << min(c, 64)) - 1)
    assert ctr.as_dict() == dict(pkts_ok=b.n, drop_sa=0, drop_format=0, drop_replay=0,
                                 drop_auth=0, drop_trailer=0, bytes_in=int(ol.sum()),
                                 bytes_out=int(b.in_len.sum()), batches=1)


def test_window_sequence_rfc4303():
    """Hand-derived RFC 4303 §3.4.3 sequence (W = 64) on one SA."""
    p = _one_sa()
    seqs = [100, 37, 36, 100, 0, 101, 38, 165, 101, 102]
    exp = [OK, OK, DREP, DREP, DREP, OK, OK, OK, DREP, OK]
    b = _packets_batch([_pk(p, q) for q in seqs], [0] * len(seqs))
    _, ol, st, ctr, win = _run(p, b)
    assert st.tolist() == exp
    top, bmp = oracle.window_state(win, 1)
    assert int(top[0]) == 165
    assert int(bmp[0]) == (1 | (1 << 63))          # 165 and 102
    assert ctr.drop_replay == 4 and ctr.pkts_ok == 6


def test_window_resumed_sa():
    """B6: an SA created with seq = s0 treats every number <= s0 as received."""
    p = _one_sa(1000)
    seqs = [1000, 937, 999, 1001, 1001, 1000 + 64, 1001 + 1]
    exp = [DREP, DREP, DREP, OK, DREP, OK, OK]
    b = _packets_batch([_pk(p, q) for q in seqs], [0] * len(seqs))
    _, _, st, _, win = _run(p, b)
    assert st.tolist() == exp
    top, bmp = oracle.window_state(win, 1)
    assert int(top[0]) == 1064
    # 1064 (bit 0), 1002 (bit 62), 1001 (bit 63)
    assert int(bmp[0]) == (1 | (1 << 62) | (1 << 63))


def test_window_is_per_batch_carried():
    """Two batches: the window state carries over between calls."""
    p = _one_sa()
    b1 = _packets_batch([_pk(p, q) for q in (1, 2, 3)], [0, 0, 0])
    b2 = _packets_batch([_pk(p, q) for q in (3, 4, 2, 70)], [0] * 4)
    _, _, st1, _, win = _run(p, b1)
    _, _, st2, _, win = _run(p, b2, win)
    assert st1.tolist() == [OK] * 3
    assert st2.tolist() == [DREP, OK, DREP, OK]


def test_trailer_padding_and_iv():
    p = _one_sa()
    P = bytes([0x45, 0x10]) + bytes(range(2, 44))          # D = 44
    good = P + bytes(range(1, 7)) + bytes([6, 4])          # p = 6 (RFC 4303 §2.4 allows up to 255)
    bad_nh = P + bytes([1, 2, 2, 41])
    bad_pad = P + bytes([1, 3, 2, 4])
    too_long = bytes(P[:18]) + bytes(range(1, 5)) + bytes([4, 4])   # D = 18 < 20
    rnd_iv = bytes.fromhex("0123456789abcdef")
    pk = [_pk(p, 1, T=good), _pk(p, 2, T=bad_nh), _pk(p, 3, T=bad_pad), _pk(p, 4, T=too_long),
          _pk(p, 5, T=good, iv=rnd_iv), _pk(p, 6, T=bad_nh + b"\x00\x00")]
    b = _packets_batch(pk, [0] * len(pk))
    out, ol, st, ctr, win = _run(p, b)
    assert st.tolist() == [OK, DTRL, DTRL, DTRL, OK, DFMT]    # last: C % 4 != 0
    for i in (0, 4):
        assert int(ol[i]) == 44 and out[b.out_off[i]:b.out_off[i] + 44].tobytes() == P
    # a trailer failure happens after the ICV check: the window still advanced
    assert int(oracle.window_state(win, 1)[0][0]) == 5
    assert ctr.drop_trailer == 3 and ctr.drop_format == 1


def test_every_single_byte_corruption_has_its_class():
    """Byte 0..23 (outer header, SPI) -> FORMAT; 24..27 (seq) -> REPLAY or AUTH;
    28.. (IV, ciphertext, ICV) -> AUTH."""
    p = _one_sa()
    base = _pk(p, 7, P=bytes([0x45, 0]) + bytes(range(2, 23)))       # D = 23, p = 3
    pk, where = [], []
    for k in range(len(base)):
        x = bytearray(base)
        x[k] ^= 0x5A
        pk.append(bytes(x))
        where.append(k)
    b = _packets_batch(pk, [0] * len(pk))
    _, _, st, _, _ = _run(p, b)
    for k, s in zip(where, st.tolist()):
        if k < 24:
            assert s == DFMT, k
        elif k < 28:
            assert s in (DREP, DAUTH), k
        else:
            assert s == DAUTH, k


def test_matches_independent_composition():
    """Mixed stream (reordering, replays, stale packets, corruption, wrong and
    invalid SA indices) over two batches: oracle == pyca/hmac/set-window
    composition packet by packet, and the final windows agree."""
    n_sa = 5
    params = gen.make_sas(n_sa, cfg_id=62)
    b, out, ol = _outbound(params, 1600, "imix", 62)
    r = gen.rng_for(62, salt=9)
    sas = oracle.make_sas(params)
    win = oracle.make_windows(sas, n_sa)
    ref = [pyca_esp.SetWindow(int(params.seq[s])) for s in range(n_sa)]
    for bi in range(2):
        order = gen.arrival_order(b.n, 900, r, reorder=6, dup=0.06, old=0.06, old_span=800)
        if bi == 1:
            order = order + 700
            order %= b.n
        ib = gen.esp_batch(out, b.out_off, ol, b.sa_idx, order, corrupt=0.04, r=r)
        sa = ib.sa_idx.copy()
        sa[::97] = n_sa + 1                      # invalid SA index
        sa[5::89] = (sa[5::89] + 1) % n_sa       # SPI mismatch
        ib.sa_idx = sa
        o2, l2, st, ctr = oracle.process_inbound(sas, win, n_sa, ib)
        for j in range(ib.n):
            s = int(ib.sa_idx[j])
            pkt = ib.in_buf[ib.in_off[j]:ib.in_off[j] + ib.in_len[j]].tobytes()
            if s >= n_sa:
                es, inner = DSA, b""
            else:
                es, inner = pyca_esp.inbound_one(int(params.spi[s]), params.aes_key[s],
                                                 params.ctr_nonce[s], params.hmac_key[s],
                                                 ref[s], pkt)
            assert int(st[j]) == es, (bi, j)
            assert int(l2[j]) == len(inner)
            assert o2[ib.out_off[j]:ib.out_off[j] + len(inner)].tobytes() == inner
        kinds = np.bincount(st, minlength=6)
        assert kinds[OK] > 0 and kinds[DREP] > 0 and kinds[DAUTH] > 0 and kinds[DFMT] > 0
        assert ctr.pkts_ok == kinds[OK] and ctr.drop_replay == kinds[DREP]
    top, bmp = oracle.window_state(win, n_sa)
    for s in range(n_sa):
        assert int(top[s]) == ref[s].top
        m = ~0 if ref[s].top >= 64 else (1 << ref[s].top) - 1    # bits of numbers >= 1
        assert int(bmp[s]) & m == ref[s].bitmap()


def test_invalid_sa_and_empty():
    p = _one_sa()
    b = _packets_batch([_pk(p, 1), _pk(p, 2)], [3, 0])
    _, ol, st, ctr, _ = _run(p, b)
    assert st.tolist() == [DSA, OK] and ol[0] == 0 and ctr.drop_sa == 1
    e = _packets_batch([], [])
    _, _, st, ctr, _ = _run(p, e)
    assert st.size == 0 and ctr.batches == 0


def test_frame_struct_sizes():
    """ctypes layouts match the C structs (16-byte window entries)."""
    import ctypes
    assert ctypes.sizeof(oracle.Replay) == 16
    assert ctypes.sizeof(oracle.InCounters) == 72
    assert struct.calcsize("!I") == 4
