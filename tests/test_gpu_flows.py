"""GPU parity for the flow -> SA lookup: the lookup kernel
against the oracle's exact-match table element by element (hits, misses,
header edge cases), and the whole path with SAs from the flow table against
the oracle's lookup followed by its sequential ESP loop."""
import struct

import numpy as np
import pytest

import oracle
from harness import assert_same, oracle_run
from paper_conf_eurosys_kimjlmsm15_b200 import gen

pytestmark = pytest.mark.gpu


def _gpu_lookup(params, flows, b):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    t = nba_ipsec.SATable(params, max_batch=max(b.n, 1))
    t.set_flow_table(flows)
    db = device.to_device(b, "cuda")
    out = torch.full((max(b.n, 1),), 7, dtype=torch.int32, device="cuda")
    t.lookup_sa(db.in_buf, db.in_off, db.in_len, out, n=b.n)
    r = out[:b.n].cpu().numpy().view(np.uint32)
    t.close()
    return r


@pytest.mark.parametrize("n_flows,miss,size", [(1, 0.0, 64), (1000, 0.1, "imix"),
                                               (65536, 0.2, 64), (200000, 0.05, 1514)])
def test_lookup_matches_oracle(n_flows, miss, size):
    n_sa = 1024
    p = gen.make_sas(n_sa, cfg_id=40)
    f = gen.make_flows(n_flows, n_sa, cfg_id=40)
    b = gen.make_batch(20000, size, n_sa, cfg_id=40)
    gen.apply_flows(b, f, cfg_id=40, miss=miss)
    exp = oracle.flow_lookup(f, b)
    assert np.array_equal(_gpu_lookup(p, f, b), exp)
    assert (exp == oracle.NO_SA).any() == (miss > 0)


def test_lookup_header_edge_cases():
    from test_oracle_flows import _batch, _flows, _ipv4
    A, B_ = 0x0A000001, 0x0A000002
    udp = struct.pack("!HHHH", 1111, 2222, 8, 0)
    pk = [_ipv4(A, B_, 17, udp), _ipv4(A, B_, 17, udp, ihl=6), _ipv4(A, B_, 17, udp, ihl=7),
          _ipv4(A, B_, 17, udp, frag=0x2000), _ipv4(A, B_, 17, udp, frag=0x0010),
          _ipv4(A, B_, 1, b"\x08\x00" * 4), _ipv4(A, B_, 6, b"\x0d\x05"),
          _ipv4(A, B_, 17, udp)[:19], _ipv4(A, B_, 17, udp, version=6),
          _ipv4(A, B_, 17, udp, ihl=15)[:40], _ipv4(B_, A, 17, udp)]
    f = _flows([(A, B_, 1111, 2222, 17, 3), (A, B_, 0, 0, 17, 4), (A, B_, 0, 0, 1, 5),
                (A, B_, 0, 0, 6, 7)])
    b = _batch(pk)
    p = gen.make_sas(8, cfg_id=41)
    assert np.array_equal(_gpu_lookup(p, f, b), oracle.flow_lookup(f, b))


def test_path_with_flow_table_sas():
    """process_batch(sa_idx=NULL): lookup + ESP path == oracle lookup + oracle ESP."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    n_sa = 256
    p = gen.make_sas(n_sa, cfg_id=42)
    f = gen.make_flows(5000, n_sa, cfg_id=42)
    bs = [gen.make_batch(8000, "imix", n_sa, cfg_id=42, batch=k) for k in range(2)]
    for k, b in enumerate(bs):
        gen.apply_flows(b, f, cfg_id=42, batch=k, miss=0.05)
        b.sa_idx = oracle.flow_lookup(f, b)            # the oracle's SAs for its own run
    t = nba_ipsec.SATable(p, max_batch=8000)
    t.set_flow_table(f)
    res = []
    for b in bs:
        db = device.to_device(b, "cuda")
        t.process(db.in_buf, db.in_off, db.in_len, None, db.out_buf, db.out_off, db.out_len, n=b.n)
        res.append(device.fetch(db))
    g = (res, t.sa_seq(), t.counters())
    t.close()
    torch.cuda.synchronize()
    assert_same(g, oracle_run(p, bs))


def test_flow_table_errors():
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    from test_oracle_flows import _flows
    p = gen.make_sas(4, cfg_id=43)
    t = nba_ipsec.SATable(p, max_batch=16)
    import torch
    z = torch.zeros(16, dtype=torch.int32, device="cuda")
    with pytest.raises(nba_ipsec.NbaIpsecError):           # no table yet
        t.lookup_sa(z, z, z, z, n=4)
    with pytest.raises(nba_ipsec.NbaIpsecError):           # no sa_idx and no table
        t.process(z, z, z, None, z, z, z, n=4)
    with pytest.raises(nba_ipsec.NbaIpsecError):           # duplicate key
        t.set_flow_table(_flows([(1, 2, 3, 4, 17, 0), (1, 2, 3, 4, 17, 1)]))
    with pytest.raises(nba_ipsec.NbaIpsecError):           # SA out of range
        t.set_flow_table(_flows([(1, 2, 3, 4, 17, 9)]))
    t.set_flow_table(_flows([(1, 2, 3, 4, 17, 1)]))
    t.set_flow_table(_flows([]))                           # removes it
    with pytest.raises(nba_ipsec.NbaIpsecError):
        t.lookup_sa(z, z, z, z, n=4)
    t.close()
