"""GPU parity for single-ingress dispatch over peer memory
(nba_ipsec_route_dispatch): routing and data movement in one pass, straight
into the owners' receive buffers.

* one process, `world` receive buffers on this GPU: every owner's packets,
  lengths, local SA indices and counts equal the numpy statement of the routing
  (tests/route_ref.py), with SA-hash and explicit owner maps, and empty batches;
* two processes on cuda:0 (the GPU box has one GPU): the owner's receive
  buffers live in ITS process and reach the ingress process through CUDA IPC
  (torch shares CUDA tensors between processes -- the same mechanism maps a
  peer GPU's memory over NVLink); each owner runs the ESP path on what it
  received, and the union equals one sequential oracle gateway."""
import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen
from route_ref import route_pack_ref

pytestmark = pytest.mark.gpu


def _read_rx(rx):
    n = int(rx.count[0].item())
    nb = int(rx.count[1].item())
    off = rx.off[:n].cpu().numpy().view(np.uint32).astype(np.int64)
    ln = rx.length[:n].cpu().numpy().view(np.uint16).astype(np.int64)
    buf = rx.buf.cpu().numpy()
    data = np.concatenate([buf[o:o + L] for o, L in zip(off, ln)]) if n else np.zeros(0, np.uint8)
    return n, nb, data, ln.astype(np.uint16), rx.sa[:n].cpu().numpy().view(np.uint32), off


@pytest.mark.parametrize("world", [1, 2, 3, 8])
@pytest.mark.parametrize("n,size,use_map", [(0, 64, False), (1, 64, False), (257, "imix", True),
                                            (20000, "imix", False), (65536, 64, True)])
def test_dispatch_matches_reference(world, n, size, use_map):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, redistribute
    n_sa_total = 300
    b = gen.make_batch(n, size, n_sa_total, cfg_id=61, layout="slots")
    if n:
        b.sa_idx[::29] = n_sa_total + 4
    sa_map = None
    if use_map:
        rng = np.random.default_rng([61, world])
        owner = rng.integers(0, world + 1, n_sa_total)
        sa_map = ((owner << 24) | rng.integers(0, 1 << 24, n_sa_total)).astype(np.uint32)
    cap_pkts, cap_bytes = max(n, 1), int(b.in_len.astype(np.int64).sum()) + 64
    rxs = [redistribute.alloc_rx(cap_pkts, cap_bytes, "cuda") for _ in range(world)]
    for r in rxs:
        r.count.fill_(-1)
    table = redistribute.rx_table(rxs, "cuda")
    db = device.to_device(b, "cuda")
    m = torch.from_numpy(sa_map.view(np.int32)).cuda() if sa_map is not None else None
    counts, nbytes = redistribute.dispatch(db, n, n_sa_total, world, table, cap_pkts, cap_bytes,
                                           sa_map=m)
    torch.cuda.synchronize()
    r_buf, r_len, r_sa, r_cnt, r_byt = route_pack_ref(b, n_sa_total, world, sa_map)
    assert counts == r_cnt and nbytes == r_byt
    c0, b0 = 0, 0
    for d in range(world):
        n_d, nb_d, data, ln, sa, off = _read_rx(rxs[d])
        assert (n_d, nb_d) == (r_cnt[d], r_byt[d])
        assert np.array_equal(ln, r_len[c0:c0 + n_d]) and np.array_equal(sa, r_sa[c0:c0 + n_d])
        assert np.array_equal(data, r_buf[b0:b0 + nb_d])
        assert np.array_equal(off, np.concatenate([[0], np.cumsum(ln.astype(np.int64))[:-1]])
                              if n_d else off)          # packed, batch order
        c0 += n_d
        b0 += nb_d


def _owner(rank, world, q_rx, q_go, q_res, n_sa_total, n):
    """Owner process (rank >= 1): allocate receive buffers, hand them to the
    ingress process (CUDA IPC), wait for the dispatch, run the path on them."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec, redistribute
    torch.cuda.set_device(0)
    cap_bytes = n * 1500 + 64
    rx = redistribute.alloc_rx(n, cap_bytes, "cuda:0")
    q_rx.put((rank, rx.buf, rx.off, rx.length, rx.sa, rx.count))
    q_go.get(timeout=300)                              # ingress stream synchronised
    res = _process_rx(rank, world, rx, n_sa_total)
    q_res.put((rank, res))
    q_go.get(timeout=300)                              # keep the tensors alive until read


def _process_rx(rank, world, rx, n_sa_total):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec, redistribute
    n, buf, off, ln, sa = redistribute.received_batch(rx)
    if n == 0:
        return []
    lens = ln[:n].to(torch.int64) & 0xFFFF
    out_off = torch.zeros(n, dtype=torch.int64, device=buf.device)
    out_off[1:] = torch.cumsum(lens[:-1] + 64, 0)
    out = torch.zeros(int((lens + 64).sum().item()) + 16, dtype=torch.uint8, device=buf.device)
    out_len = torch.zeros(n, dtype=torch.int16, device=buf.device)
    params = gen.make_sas(n_sa_total // world, cfg_id=62, rank=rank, world=world)
    with nba_ipsec.SATable(params, device=0, max_batch=n) as t:
        t.process(buf, off, ln, sa, out, out_off.to(torch.int32), out_len, n=n)
        torch.cuda.synchronize()
    o = out.cpu().numpy()
    oo = out_off.cpu().numpy()
    ol = out_len.cpu().numpy().view(np.uint16)
    return [o[oo[j]:oo[j] + ol[j]].tobytes() for j in range(n)]


def test_dispatch_two_processes_ipc_union_equals_one_gateway():
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, redistribute
    world, n_sa_total, n = 2, 16, 3000
    ctx = mp.get_context("spawn")
    q_rx, q_go, q_res = ctx.Queue(), ctx.Queue(), ctx.Queue()
    p = ctx.Process(target=_owner, args=(1, world, q_rx, q_go, q_res, n_sa_total, n))
    p.start()
    try:
        torch.cuda.set_device(0)
        b = gen.make_batch(n, "imix", n_sa_total, cfg_id=62, layout="packed")
        b.sa_idx[::41] = n_sa_total + 2
        own = redistribute.alloc_rx(n, n * 1500 + 64, "cuda:0")
        r, *t1 = q_rx.get(timeout=300)                  # owner 1's buffers, IPC-mapped here
        peer = redistribute.PeerRx(*t1)
        table = redistribute.rx_table([own, peer], "cuda:0")
        db = device.to_device(b, "cuda:0")
        counts, _ = redistribute.dispatch(db, n, n_sa_total, world, table, n, n * 1500 + 64)
        torch.cuda.synchronize()
        q_go.put(1)
        mine = _process_rx(0, world, own, n_sa_total)
        r1, theirs = q_res.get(timeout=300)
        q_go.put(1)
        p.join(timeout=120)
        assert p.exitcode == 0
    finally:
        if p.is_alive():
            p.kill()
    assert counts == [len(mine), len(theirs)]
    parts = [gen.make_sas(n_sa_total // world, cfg_id=62, rank=r, world=world) for r in range(world)]
    fields = ["spi", "tunnel_src", "tunnel_dst", "aes_key", "ctr_nonce", "hmac_key", "seq"]
    allp = gen.SAParams(*[np.stack([getattr(parts[s % world], f)[s // world] for s in range(n_sa_total)])
                          for f in fields])
    ref_out, ref_len, _ = oracle.process_batch(oracle.make_sas(allp), n_sa_total, b)
    got = {0: mine, 1: theirs}
    seen = {0: 0, 1: 0}
    for i in range(b.n):
        s = int(b.sa_idx[i])
        if s >= n_sa_total:
            continue
        d = s % world
        assert got[d][seen[d]] == ref_out[b.out_off[i]:b.out_off[i] + ref_len[i]].tobytes()
        seen[d] += 1
    assert seen == {0: len(mine), 1: len(theirs)}


@pytest.mark.parametrize("cap_pkts_frac,cap_bytes_frac", [(1.0, 0.37), (0.5, 1.0), (0.6, 0.4),
                                                          (1.0, 0.0)])
def test_dispatch_capacity_overflow(cap_pkts_frac, cap_bytes_frac):
    """Receive buffers smaller than an owner's share: the owner gets exactly the
    longest prefix of its packets (batch order) that fits both capacities, its
    published count says so (no stale entries past it), nothing is written past
    the capacity, and dest_counts / dest_bytes still report the full routing."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, redistribute
    n, n_sa_total, world = 3000, 40, 2
    b = gen.make_batch(n, "imix", n_sa_total, cfg_id=62, layout="slots")
    r_buf, r_len, r_sa, r_cnt, r_byt = route_pack_ref(b, n_sa_total, world)
    cap_pkts = int(min(r_cnt) * cap_pkts_frac)
    cap_bytes = int(min(r_byt) * cap_bytes_frac)
    guard = 4096
    rxs = [redistribute.alloc_rx(cap_pkts + guard, cap_bytes + guard, "cuda") for _ in range(world)]
    for r in rxs:
        r.buf.fill_(0x5A)
        r.count.fill_(-1)
    table = redistribute.rx_table(rxs, "cuda")
    db = device.to_device(b, "cuda")
    counts, nbytes = redistribute.dispatch(db, n, n_sa_total, world, table, cap_pkts, cap_bytes)
    torch.cuda.synchronize()
    assert counts == r_cnt and nbytes == r_byt
    c0, b0 = 0, 0
    for d in range(world):
        ln_all = r_len[c0:c0 + r_cnt[d]].astype(np.int64)
        ends = np.cumsum(ln_all)
        fit = int(np.sum((np.arange(r_cnt[d]) < cap_pkts) & (ends <= cap_bytes)))
        n_d, nb_d, data, ln, sa, off = _read_rx(rxs[d])
        assert (n_d, nb_d) == (fit, int(ends[fit - 1]) if fit else 0)
        assert np.array_equal(ln, r_len[c0:c0 + fit]) and np.array_equal(sa, r_sa[c0:c0 + fit])
        assert np.array_equal(data, r_buf[b0:b0 + nb_d])
        tail = rxs[d].buf[cap_bytes:].cpu().numpy()
        assert np.all(tail == 0x5A), "bytes written past cap_bytes"
        c0 += r_cnt[d]
        b0 += r_byt[d]
