"""Single-ingress redistribution across 2 and 3 processes on
gloo (CPU): rank 0 receives all the traffic, routes it by SA owner (numpy
statement of the routing, tests/route_ref.py), the exchange moves it with
all-to-alls, every owner runs the oracle on its own SA shard, and the union of
the owners' outputs equals ONE sequential oracle run over the whole stream."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_eurosys_kimjlmsm15_b200 import gen


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist

    import oracle
    from paper_conf_eurosys_kimjlmsm15_b200 import redistribute
    from route_ref import packed_cpu
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n_sa_total = 12
    b = gen.make_batch(900, "imix", n_sa_total, cfg_id=88, layout="packed")
    b.sa_idx[::37] = n_sa_total + 5                          # not routable
    if rank == 0:
        p = packed_cpu(b, n_sa_total, world)
    else:                                                    # no ingress traffic here
        empty = gen.make_batch(0, 64, n_sa_total, cfg_id=88, layout="packed")
        p = packed_cpu(empty, n_sa_total, world)
    r = redistribute.exchange(p)
    n = r.n
    lens = r.in_len[:n].numpy().view(np.uint16).astype(np.int64)
    out_off = np.concatenate([[0], np.cumsum(lens + 64)[:-1]]) if n else np.zeros(0, np.int64)
    mine = gen.Batch(n=n, in_buf=r.in_buf.numpy(), in_off=r.in_off[:n].numpy().view(np.uint32),
                     in_len=lens.astype(np.uint16), sa_idx=r.sa_idx[:n].numpy().view(np.uint32),
                     out_off=out_off.astype(np.uint32), out_pool_bytes=int((lens + 64).sum()) + 16,
                     frame_len=(lens + 14).astype(np.uint32))
    params = gen.make_sas(n_sa_total // world, cfg_id=88, rank=rank, world=world)
    out, ol, ctr = oracle.process_batch(oracle.make_sas(params), len(params.spi), mine)
    res = [out[mine.out_off[j]:mine.out_off[j] + ol[j]].tobytes() for j in range(n)]
    q.put((rank, res, ctr.as_dict()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_single_ingress_union_equals_one_gateway(world):
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    got = dict((r, (res, c)) for r, res, c in (q.get(timeout=180) for _ in range(world)))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    n_sa_total = 12
    b = gen.make_batch(900, "imix", n_sa_total, cfg_id=88, layout="packed")
    b.sa_idx[::37] = n_sa_total + 5
    # one gateway with all SAs: global SA s has the parameters of (rank s % world, j = s // world)
    parts = [gen.make_sas(n_sa_total // world, cfg_id=88, rank=r, world=world) for r in range(world)]
    fields = ["spi", "tunnel_src", "tunnel_dst", "aes_key", "ctr_nonce", "hmac_key", "seq"]
    allp = gen.SAParams(*[np.stack([getattr(parts[s % world], f)[s // world] for s in range(n_sa_total)])
                          for f in fields])
    ref_out, ref_len, ref_ctr = oracle.process_batch(oracle.make_sas(allp), n_sa_total, b)
    seen = {r: 0 for r in range(world)}
    for i in range(b.n):
        s = int(b.sa_idx[i])
        if s >= n_sa_total:
            assert int(ref_len[i]) == 0
            continue
        r = s % world
        res, _ = got[r]
        assert res[seen[r]] == ref_out[b.out_off[i]:b.out_off[i] + ref_len[i]].tobytes()
        seen[r] += 1
    assert sum(seen.values()) == sum(len(got[r][0]) for r in range(world))
    assert sum(got[r][1]["pkts_ok"] for r in range(world)) == ref_ctr.pkts_ok
