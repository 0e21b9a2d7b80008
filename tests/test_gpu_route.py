"""GPU parity for single-ingress routing: the route/pack
kernels against the numpy statement of the routing (tests/route_ref.py),
array by array, and a one-GPU stand-in for the exchange (each destination's
slice processed on that owner's SA table) against one sequential oracle
gateway with all SAs."""
import numpy as np
import pytest

import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen
from route_ref import route_pack_ref

pytestmark = pytest.mark.gpu


def _gpu_pack(b, n_sa_total, world):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, redistribute
    db = device.to_device(b, "cuda")
    p = redistribute.pack(db, b.n, n_sa_total, world)
    torch.cuda.synchronize()
    n_in, b_in = sum(p.counts), sum(p.nbytes)
    return (p.buf[:b_in].cpu().numpy(), p.length[:n_in].cpu().numpy().view(np.uint16),
            p.sa[:n_in].cpu().numpy().view(np.uint32), p.counts, p.nbytes)


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("n,size", [(1, 64), (255, "imix"), (257, 1514), (20000, "imix")])
def test_pack_matches_reference(world, n, size):
    n_sa_total = 40
    b = gen.make_batch(n, size, n_sa_total, cfg_id=31, layout="packed")
    b.sa_idx[::29] = n_sa_total + 1
    g = _gpu_pack(b, n_sa_total, world)
    r = route_pack_ref(b, n_sa_total, world)
    assert g[3] == r[3] and g[4] == r[4]
    assert np.array_equal(g[1], r[1]) and np.array_equal(g[2], r[2])
    assert np.array_equal(g[0], r[0])


def test_one_gpu_exchange_stand_in_equals_one_gateway():
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    import torch
    world, n_sa_total = 4, 64
    b = gen.make_batch(30000, "imix", n_sa_total, cfg_id=32, layout="packed")
    buf, lens, sas, counts, nbytes = _gpu_pack(b, n_sa_total, world)
    parts = [gen.make_sas(n_sa_total // world, cfg_id=32, rank=r, world=world) for r in range(world)]
    fields = ["spi", "tunnel_src", "tunnel_dst", "aes_key", "ctr_nonce", "hmac_key", "seq"]
    allp = gen.SAParams(*[np.stack([getattr(parts[s % world], f)[s // world] for s in range(n_sa_total)])
                          for f in fields])
    ref_out, ref_len, _ = oracle.process_batch(oracle.make_sas(allp), n_sa_total, b)
    c0, b0 = 0, 0
    for d in range(world):
        n = counts[d]
        L = lens[c0:c0 + n].astype(np.int64)
        in_off = np.concatenate([[0], np.cumsum(L)[:-1]]).astype(np.uint32)
        out_off = np.concatenate([[0], np.cumsum(L + 64)[:-1]]).astype(np.uint32)
        mine = gen.Batch(n=n, in_buf=buf[b0:b0 + nbytes[d]].copy(), in_off=in_off,
                         in_len=L.astype(np.uint16), sa_idx=sas[c0:c0 + n].copy(), out_off=out_off,
                         out_pool_bytes=int((L + 64).sum()) + 16, frame_len=(L + 14).astype(np.uint32))
        from harness import gpu_run
        (res,), _, _ = gpu_run(parts[d], [mine])
        out, ol = res
        idx = np.nonzero(b.sa_idx % world == d)[0]
        for j, i in enumerate(idx):
            assert out[out_off[j]:out_off[j] + ol[j]].tobytes() == \
                ref_out[b.out_off[i]:b.out_off[i] + ref_len[i]].tobytes()
        c0 += n
        b0 += nbytes[d]
    torch.cuda.synchronize()
