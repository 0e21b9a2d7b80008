"""Adaptive split across 2 and 3 processes on gloo (readings
L6/L7): rank 0 receives all traffic; between batches the SA ownership changes
(owner maps from the library's nba_ipsec_alb_assign for a scripted sequence of
node steps, including "everything on one device"), the counters of the SAs
that move are handed over with alb.handover_dist (MAX all-reduce), packets are
routed by the map (numpy statement, tests/route_ref.py) and exchanged with the
all-to-alls, and every rank runs the oracle on what it owns.  The union over
ranks and batches equals ONE sequential oracle gateway over the whole stream."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_eurosys_kimjlmsm15_b200 import gen

N_SA = 16
K = 25
# node steps per batch (heap order, root first): moves SAs back and forth
SCHEDULE = {2: [[12], [20], [0], [25], [7]],
            3: [[12, 0, 12], [3, 0, 25], [25, 0, 0], [0, 0, 12], [16, 0, 5]]}


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _batches():
    out = []
    for j in range(len(SCHEDULE[2])):
        b = gen.make_batch(300, "imix", N_SA, cfg_id=91, batch=j, layout="packed")
        b.sa_idx[::41] = N_SA + 3                    # not routable
        out.append(b)
    return out


class OracleTable:
    """Stand-in for one device's SA table (all SAs; the owner's counter is live)."""

    def __init__(self, params):
        import oracle
        self.sas = oracle.make_sas(params)

    def sa_seq(self, stream=None):
        import oracle
        return oracle.sa_seq(self.sas, N_SA)

    def write_sa_seq(self, seq, stream=None):
        for s in range(N_SA):
            self.sas[s].seq = int(seq[s])


def _worker(rank, world, port, q):
    import torch.distributed as dist

    import oracle
    from paper_conf_eurosys_kimjlmsm15_b200 import alb, nba_ipsec, redistribute
    from route_ref import packed_cpu
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    params = gen.make_sas(N_SA, cfg_id=91)
    table = OracleTable(params)
    old_owner = None
    results = []
    for j, b in enumerate(_batches()):
        owner, sa_map = nba_ipsec.alb_assign(N_SA, world, SCHEDULE[world][j], K)
        if old_owner is not None:
            alb.handover_dist(table, old_owner, rank)
        old_owner = owner
        if rank == 0:
            p = packed_cpu(b, N_SA, world, sa_map)
        else:
            empty = gen.make_batch(0, 64, N_SA, cfg_id=91, layout="packed")
            p = packed_cpu(empty, N_SA, world, sa_map)
        r = redistribute.exchange(p)
        n = r.n
        lens = r.in_len[:n].numpy().view(np.uint16).astype(np.int64)
        out_off = np.concatenate([[0], np.cumsum(lens + 64)[:-1]]) if n else np.zeros(0, np.int64)
        mine = gen.Batch(n=n, in_buf=r.in_buf.numpy(), in_off=r.in_off[:n].numpy().view(np.uint32),
                         in_len=lens.astype(np.uint16), sa_idx=r.sa_idx[:n].numpy().view(np.uint32),
                         out_off=out_off.astype(np.uint32), out_pool_bytes=int((lens + 64).sum()) + 16,
                         frame_len=(lens + 14).astype(np.uint32))
        out, ol, ctr = oracle.process_batch(table.sas, N_SA, mine)
        results.append(([out[mine.out_off[i]:mine.out_off[i] + ol[i]].tobytes() for i in range(n)],
                         ctr.as_dict()["pkts_ok"]))
    q.put((rank, results, table.sa_seq(), old_owner))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_adaptive_split_union_equals_one_gateway(world):
    import oracle
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    got = {}
    for _ in range(world):
        r, res, seq, last_owner = q.get(timeout=240)
        got[r] = (res, seq, last_owner)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    ref = oracle.make_sas(gen.make_sas(N_SA, cfg_id=91))
    moved = 0
    prev = None
    for j, b in enumerate(_batches()):
        owner, _ = nba_ipsec.alb_assign(N_SA, world, SCHEDULE[world][j], K)
        if prev is not None:
            moved += int((owner != prev).sum())
        prev = owner
        ref_out, ref_len, ref_ctr = oracle.process_batch(ref, N_SA, b)
        seen = {r: 0 for r in range(world)}
        for i in range(b.n):
            s = int(b.sa_idx[i])
            if s >= N_SA:
                assert int(ref_len[i]) == 0
                continue
            r = int(owner[s])
            res = got[r][0][j][0]
            assert res[seen[r]] == ref_out[b.out_off[i]:b.out_off[i] + ref_len[i]].tobytes()
            seen[r] += 1
        assert all(seen[r] == len(got[r][0][j][0]) for r in range(world))
        assert sum(got[r][0][j][1] for r in range(world)) == ref_ctr.pkts_ok
    assert moved >= N_SA                               # SAs really changed owners
    # the live counters (each on its last owner) equal the single gateway's
    live = np.zeros(N_SA, np.uint32)
    for r in range(world):
        m = got[r][2] == r
        live[m] = got[r][1][m]
    assert np.array_equal(live, oracle.sa_seq(ref, N_SA))
