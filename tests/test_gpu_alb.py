"""GPU parity for the adaptive split: routing by an owner map
(nba_ipsec_route_pack_map) against the numpy statement (tests/route_ref.py),
the counter hand-over (nba_ipsec_write_sa_seq) against the oracle started from
the same counters, and two SA tables on one GPU standing in for two devices
while the library's controller/assignment move SAs between them: the union of
their outputs over consecutive batches equals ONE sequential oracle gateway."""
import numpy as np
import pytest

import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen
from route_ref import route_pack_ref

pytestmark = pytest.mark.gpu


def _gpu_pack_map(b, n_sa_total, world, sa_map):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, redistribute
    db = device.to_device(b, "cuda")
    m = torch.from_numpy(np.asarray(sa_map, np.uint32).view(np.int32)).cuda()
    p = redistribute.pack(db, b.n, n_sa_total, world, sa_map=m)
    torch.cuda.synchronize()
    n_in, b_in = sum(p.counts), sum(p.nbytes)
    return (p.buf[:b_in].cpu().numpy(), p.length[:n_in].cpu().numpy().view(np.uint16),
            p.sa[:n_in].cpu().numpy().view(np.uint32), p.counts, p.nbytes)


@pytest.mark.parametrize("world", [1, 2, 5, 8])
@pytest.mark.parametrize("n,size", [(1, 64), (257, "imix"), (20000, "imix")])
def test_pack_map_matches_reference(world, n, size):
    n_sa_total = 300
    rng = np.random.default_rng([7, world, n])
    owner = rng.integers(0, world + 1, n_sa_total)            # owner == world: not sent
    local = rng.integers(0, 1 << 24, n_sa_total)
    sa_map = ((owner << 24) | local).astype(np.uint32)
    b = gen.make_batch(n, size, n_sa_total, cfg_id=33, layout="packed")
    b.sa_idx[::31] = n_sa_total + 2
    g = _gpu_pack_map(b, n_sa_total, world, sa_map)
    r = route_pack_ref(b, n_sa_total, world, sa_map)
    assert g[3] == r[3] and g[4] == r[4]
    assert np.array_equal(g[1], r[1]) and np.array_equal(g[2], r[2])
    assert np.array_equal(g[0], r[0])


def test_write_sa_seq_then_process_matches_oracle():
    from harness import assert_same, gpu_run, oracle_run
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    n_sa = 64
    p = gen.make_sas(n_sa, cfg_id=34)
    b = [gen.make_batch(5000, "imix", n_sa, cfg_id=34, batch=j) for j in range(2)]
    seq = np.random.default_rng(34).integers(0, 1 << 31, n_sa).astype(np.uint32)
    seq[:4] = [0xFFFFFFFF, 0xFFFFFFFE, 0xFFFFFF00, 0]          # exhausted / overflowing SAs
    with nba_ipsec.SATable(p, device=0, max_batch=5000) as t:
        t.write_sa_seq(seq)
        assert np.array_equal(t.sa_seq(), seq)
        got = gpu_run(p, b, table=t)
    p2 = gen.SAParams(*[getattr(p, f) for f in ("spi", "tunnel_src", "tunnel_dst", "aes_key",
                                                "ctr_nonce", "hmac_key")], seq=seq)
    assert_same(got, oracle_run(p2, b))


def test_two_tables_adaptive_split_equals_one_gateway():
    """Device d = its own SA table + stream on cuda:0.  Every step: the ingress
    batch is routed by the current owner map on the GPU, each table processes
    its share, the library controller observes the step, and when the owner map
    changes the counters of the moved SAs are handed over before the next step."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import alb, device, nba_ipsec, redistribute
    n_sa, n, steps_run = 128, 6000, 14
    p = gen.make_sas(n_sa, cfg_id=35)
    bal = alb.Balancer(n_sa, 2, steps=8, init_step=4, history=4, update_ns=1, wait_min=0,
                       wait_max=1)
    tables = [nba_ipsec.SATable(p, device=0, max_batch=n) for _ in range(2)]
    streams = [torch.cuda.Stream() for _ in range(2)]
    ref = oracle.make_sas(p)
    owner, sa_map = bal.assignment()
    maps_seen, t_ns = set(), 0
    try:
        for j in range(steps_run):
            b = gen.make_batch(n, "imix", n_sa, cfg_id=35, batch=j, layout="packed")
            ref_out, ref_len, _ = oracle.process_batch(ref, n_sa, b)
            db = device.to_device(b, "cuda")
            m = torch.from_numpy(sa_map.view(np.int32)).cuda()
            pk = redistribute.pack(db, n, n_sa, 2, sa_map=m)
            maps_seen.add(tuple(np.bincount(owner, minlength=2)))
            c0, b0, dts, pk_n = 0, 0, [], []
            for d in range(2):
                cnt, nb = pk.counts[d], pk.nbytes[d]
                L = pk.length[c0:c0 + cnt].to(torch.int64) & 0xFFFF
                in_off = torch.zeros(max(cnt, 1), dtype=torch.int64, device="cuda")
                if cnt > 1:
                    in_off[1:cnt] = torch.cumsum(L[:-1], 0)
                in_off = (in_off + b0).to(torch.int32)
                out_off = torch.zeros(max(cnt, 1), dtype=torch.int64, device="cuda")
                if cnt > 1:
                    out_off[1:cnt] = torch.cumsum(L[:-1] + 64, 0)
                out_off = out_off.to(torch.int32)
                out_buf = torch.zeros(int((L + 64).sum().item()) + 16 if cnt else 16,
                                      dtype=torch.uint8, device="cuda")
                out_len = torch.zeros(max(cnt, 1), dtype=torch.int16, device="cuda")
                ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                streams[d].wait_stream(torch.cuda.current_stream())
                with torch.cuda.stream(streams[d]):
                    ev0.record(streams[d])
                    tables[d].process(pk.buf, in_off, pk.length[c0:], pk.sa[c0:], out_buf, out_off,
                                      out_len, n=cnt, stream=streams[d])
                    ev1.record(streams[d])
                streams[d].synchronize()
                dts.append(int(ev0.elapsed_time(ev1) * 1e6))
                pk_n.append(cnt)
                got_len = out_len[:cnt].cpu().numpy().view(np.uint16)
                got = out_buf.cpu().numpy()
                oo = out_off[:cnt].cpu().numpy()
                idx = np.nonzero((b.sa_idx < n_sa) & (owner[np.minimum(b.sa_idx, n_sa - 1)] == d))[0]
                assert idx.size == cnt
                for k, i in enumerate(idx):
                    assert got_len[k] == ref_len[i]
                    assert got[oo[k]:oo[k] + got_len[k]].tobytes() == \
                        ref_out[b.out_off[i]:b.out_off[i] + ref_len[i]].tobytes()
                c0 += cnt
                b0 += nb
            t_ns += max(dts) + 1
            # step j's sample; the next step uses the (possibly) new split
            if bal.observe(t_ns, dts, pk_n):
                new_owner, new_map = bal.assignment()
                alb.handover_tables(tables, owner, new_owner)
                owner, sa_map = new_owner, new_map
        live = np.where(owner == 0, tables[0].sa_seq(), tables[1].sa_seq())
        assert np.array_equal(live, oracle.sa_seq(ref, n_sa))
        assert len(maps_seen) >= 3                       # the split really moved
    finally:
        for t in tables:
            t.close()
