"""Pins for the oracle's flow -> SA lookup (readings F1..F4 in
DESIGN.md): agreement with the generator's own flow assignment (ground truth by
construction), an independent Python dict implementation on hand-made edge
cases (IP options, fragments, portless protocols, truncated headers, IPv6),
and duplicate-key rejection.  None of these values come from the CUDA path."""
import struct

import numpy as np
import pytest

import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen

NO_SA = 0xFFFFFFFF


def _ipv4(src, dst, proto, payload, ihl=5, frag=0, version=4):
    opts = b"\x01" * (4 * (ihl - 5))
    tot = 4 * ihl + len(payload)
    h = struct.pack("!BBHHHBBHII", (version << 4) | ihl, 0, tot, 7, frag, 64, proto, 0, src, dst)
    return h + opts + payload


def _batch(pkts, n_sa=8):
    n = len(pkts)
    lens = np.array([len(p) for p in pkts], np.int64)
    off = np.concatenate([[0], np.cumsum(lens)[:-1]]).astype(np.uint32)
    buf = np.zeros(int(lens.sum()) + 16, np.uint8)
    for i, p in enumerate(pkts):
        buf[off[i]:off[i] + len(p)] = np.frombuffer(p, np.uint8)
    return gen.Batch(n=n, in_buf=buf, in_off=off, in_len=lens.astype(np.uint16),
                     sa_idx=np.zeros(n, np.uint32), out_off=off.copy(),
                     out_pool_bytes=int(buf.size), frame_len=(lens + 14).astype(np.uint32))


def _py_key(P):
    """Independent restatement of F1/F2 (Python)."""
    if len(P) < 20 or P[0] >> 4 != 4 or (P[0] & 15) < 5 or len(P) < 4 * (P[0] & 15):
        return None
    ihl = P[0] & 15
    src, dst = struct.unpack("!II", P[12:20])
    proto = P[9]
    frag = struct.unpack("!H", P[6:8])[0] & 0x1FFF
    sp = dp = 0
    if proto in (6, 17) and frag == 0 and len(P) >= 4 * ihl + 4:
        sp, dp = struct.unpack("!HH", P[4 * ihl:4 * ihl + 4])
    return (src, dst, proto, sp, dp)


def _flows(rows):
    a = np.array(rows, np.int64).reshape(-1, 6) if rows else np.zeros((0, 6), np.int64)
    return gen.Flows(src=a[:, 0].astype(np.uint32), dst=a[:, 1].astype(np.uint32),
                     sport=a[:, 2].astype(np.uint16), dport=a[:, 3].astype(np.uint16),
                     proto=a[:, 4].astype(np.uint8), sa=a[:, 5].astype(np.uint32))


def test_generated_flows_ground_truth():
    for n_flows, miss in ((1, 0.0), (1000, 0.1), (20000, 0.3)):
        f = gen.make_flows(n_flows, 64, cfg_id=7)
        b = gen.make_batch(3000, "imix", 64, cfg_id=7)
        fi = gen.apply_flows(b, f, cfg_id=7, miss=miss)
        exp = np.where(fi >= 0, f.sa[np.maximum(fi, 0)], NO_SA).astype(np.uint32)
        assert np.array_equal(oracle.flow_lookup(f, b), exp)


def test_header_edge_cases_vs_python():
    A, B_ = 0x0A000001, 0x0A000002
    udp = struct.pack("!HHHH", 1111, 2222, 8, 0)
    tcp = struct.pack("!HH", 3333, 4444) + b"\x00" * 16
    pk = [
        _ipv4(A, B_, 17, udp),                       # plain UDP
        _ipv4(A, B_, 17, udp, ihl=6),                # options: ports after 24 bytes
        _ipv4(A, B_, 17, udp, frag=0x2000),          # first fragment (MF, offset 0): ports used
        _ipv4(A, B_, 17, udp, frag=0x0010),          # later fragment: ports 0
        _ipv4(A, B_, 1, b"\x08\x00" * 4),            # ICMP: no ports
        _ipv4(A, B_, 6, tcp),                        # TCP
        _ipv4(A, B_, 6, b"\x0d\x05"),                # TCP with 2 bytes after the header: ports 0
        _ipv4(A, B_, 17, udp)[:19],                  # shorter than an IPv4 header
        _ipv4(A, B_, 17, udp, version=6),            # not IPv4
        _ipv4(A, B_, 17, udp, ihl=15)[:40],          # IHL beyond the datagram
        _ipv4(B_, A, 17, udp),                       # reverse direction: another flow
    ]
    rows = [(A, B_, 1111, 2222, 17, 3), (A, B_, 0, 0, 17, 4), (A, B_, 0, 0, 1, 5),
            (A, B_, 3333, 4444, 6, 6), (A, B_, 0, 0, 6, 7)]
    f = _flows(rows)
    table = {(r[0], r[1], r[4], r[2], r[3]): r[5] for r in rows}
    exp = [table.get(_py_key(p), NO_SA) if _py_key(p) else NO_SA for p in pk]
    got = oracle.flow_lookup(f, _batch(pk)).tolist()
    assert got == exp
    assert got == [3, 3, 3, 4, 5, 6, 7, NO_SA, NO_SA, NO_SA, NO_SA]


def test_duplicate_keys_rejected():
    f = _flows([(1, 2, 3, 4, 17, 0), (1, 2, 3, 4, 17, 1)])
    with pytest.raises(ValueError):
        oracle.flow_lookup(f, _batch([_ipv4(1, 2, 17, b"\x00" * 8)]))
