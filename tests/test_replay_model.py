"""Host-side check of the batch-parallel anti-replay decision used by the CUDA
inbound path (k_in_replay.cu / k_in_decide): written in numpy as
    top_j  = max(top_0, prefix-max of q over earlier authenticated packets of the SA)
    pass_j = q != 0 and (q > top_j or (top_j - q < 64 and q not marked at batch
             start and no earlier authenticated packet of the SA has the same q))
and compared with the sequential oracle (RFC 4303 §3.4.3 one packet at a time)
on streams full of reordering, duplicates, stale packets and forgeries.  Format
and ICV validity come from the independent pyca/hmac composition."""
import hashlib
import hmac
import struct

import numpy as np
import pytest

import oracle
import pyca_esp
from paper_conf_eurosys_kimjlmsm15_b200 import gen

W = 64


def _flags(params, b):
    """(fmt_ok, icv_ok, q) per packet, independent of the oracle."""
    n_sa = len(params.spi)
    fmt = np.zeros(b.n, bool)
    icv = np.zeros(b.n, bool)
    q = np.zeros(b.n, np.int64)
    for j in range(b.n):
        s = int(b.sa_idx[j])
        pkt = b.in_buf[b.in_off[j]:b.in_off[j] + b.in_len[j]].tobytes()
        L = len(pkt)
        if s >= n_sa or L < 72 or L > 1552 or (L - 48) % 4:
            continue
        if pkt[0] != 0x45 or pkt[9] != 50 or struct.unpack("!H", pkt[2:4])[0] != L:
            continue
        if struct.unpack("!H", pkt[6:8])[0] & 0x3FFF or pyca_esp.csum(pkt[:20]) != 0:
            continue
        if struct.unpack("!I", pkt[20:24])[0] != int(params.spi[s]):
            continue
        fmt[j] = True
        q[j] = struct.unpack("!I", pkt[24:28])[0]
        mac = hmac.new(bytes(params.hmac_key[s]), pkt[20:L - 12], hashlib.sha1).digest()[:12]
        icv[j] = mac == pkt[L - 12:]
    return fmt, icv, q


def _parallel_decide(sa, fmt, icv, q, top0, bmp0):
    n = len(sa)
    A = fmt & icv
    passed = np.zeros(n, bool)
    first = {}                                  # (s, q) -> smallest index in A
    for j in np.nonzero(A)[0]:
        first.setdefault((int(sa[j]), int(q[j])), int(j))
    run = {}                                    # running max per SA (prefix max)
    for j in range(n):
        if not fmt[j]:
            continue
        s, x = int(sa[j]), int(q[j])
        tj = max(int(top0[s]), run.get(s, 0))
        t0, b0 = int(top0[s]), int(bmp0[s])
        ok = x != 0
        if ok and x <= tj:
            if tj - x >= W:
                ok = False
            elif x <= t0 and (b0 >> (t0 - x)) & 1:
                ok = False
            elif first.get((s, x), n) < j:
                ok = False
        passed[j] = ok
        if A[j]:
            run[s] = max(run.get(s, 0), x)
    return passed


@pytest.mark.parametrize("n_sa,seq0", [(1, 0), (3, 0), (7, 50), (16, 0)])
def test_parallel_replay_rule_equals_sequential(n_sa, seq0):
    p = gen.make_sas(n_sa, cfg_id=80 + n_sa)
    b0 = gen.make_batch(1500, "imix", n_sa, cfg_id=80 + n_sa)
    sas_out = oracle.make_sas(p)
    out, ol, _ = oracle.process_batch(sas_out, n_sa, b0)
    q_params = p.copy()
    q_params.seq[:] = seq0
    sas = oracle.make_sas(q_params)
    win = oracle.make_windows(sas, n_sa)
    r = gen.rng_for(80 + n_sa, salt=4)
    start = 0
    for k in range(3):
        order = (gen.arrival_order(b0.n, 600, r, reorder=8, dup=0.08, old=0.08, old_span=900)
                 + start) % b0.n
        start += 500
        b = gen.esp_batch(out, b0.out_off, ol, b0.sa_idx, order, corrupt=0.05, r=r)
        top0, bmp0 = oracle.window_state(win, n_sa)
        fmt, icv, q = _flags(p, b)
        passed = _parallel_decide(b.sa_idx, fmt, icv, q, top0, bmp0)
        _, _, st, _ = oracle.process_inbound(sas, win, n_sa, b)
        exp_replay = fmt & ~passed
        assert np.array_equal(st == oracle.IN_DROP_REPLAY, exp_replay)
        assert np.array_equal(st == oracle.IN_DROP_AUTH, fmt & passed & ~icv)
        # window after the batch: edge = max(top0, max over A), bits = shifted
        # start bitmap | accepted numbers
        top1, bmp1 = oracle.window_state(win, n_sa)
        for s in range(n_sa):
            mA = (b.sa_idx == s) & fmt & icv
            t1 = max(int(top0[s]), int(q[mA].max()) if mA.any() else 0)
            assert int(top1[s]) == t1
            sh = t1 - int(top0[s])
            bits = 0 if sh >= W else (int(bmp0[s]) << sh) & ((1 << 64) - 1)
            for j in np.nonzero(mA & passed)[0]:
                if t1 - int(q[j]) < W:
                    bits |= 1 << (t1 - int(q[j]))
            assert int(bmp1[s]) == bits
