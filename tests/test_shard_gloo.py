"""Multi-GPU host logic on CPU (world_size 2, gloo): SA-hash sharding gives each
rank a disjoint SA set, per-rank streams are independent (no data-path
collective), and the end-of-run reductions (SUM of counters, MAX of elapsed
time) are what bench.py reports.  Each rank runs the oracle on its shard; the
union of the shards must equal one oracle run over the concatenated traffic."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_eurosys_kimjlmsm15_b200 import gen, shard


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n_sa_total, n, out_q):
    import torch.distributed as dist

    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    p, b = shard.rank_workload(9, n, "imix", n_sa_total, rank, world)
    sas = oracle.make_sas(p)
    out, ol, ctr = oracle.process_batch(sas, len(p.spi), b, n_threads=1)
    red = shard.reduce_counters(ctr.as_dict())
    mx = shard.max_over_ranks(float(rank + 1) * 1.5)
    out_q.put((rank, p.spi.tolist(), ctr.as_dict(), red, mx))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_gloo_reduce_and_disjoint_shards():
    world, n_sa_total, n = 2, 16, 600
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n_sa_total, n, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    res.sort()
    spis = [set(r[1]) for r in res]
    assert spis[0].isdisjoint(spis[1])
    assert spis[0] | spis[1] == {0x100 + s for s in range(n_sa_total)}
    for rank, spi, _, _, _ in res:     # global SA id s = rank + world * j
        assert all((x - 0x100) % world == rank for x in spi)
    total = {k: sum(r[2][k] for r in res) for k in shard.COUNTER_KEYS}
    for r in res:
        assert r[3] == total                 # SUM all-reduce
        assert r[4] == pytest.approx(3.0)    # MAX all-reduce


def test_virtual_shard_union_equals_single_oracle_cpu():
    """shard_batch: splitting one batch by s mod G and running each shard on its
    own SA table reproduces the single sequential oracle run byte for byte."""
    import oracle
    n_sa, n = 24, 900
    p = gen.make_sas(n_sa, cfg_id=57)
    b = gen.make_batch(n, "imix", n_sa, cfg_id=57)
    b.sa_idx[::50] = n_sa + 3           # some invalid SAs
    ref_out, ref_len, ref_ctr = oracle.process_batch(oracle.make_sas(p), n_sa, b)
    for G in (2, 3, 4):
        tot = dict.fromkeys(shard.COUNTER_KEYS, 0)
        seen = np.zeros(n, bool)
        for r in range(G):
            sp, sb, idx = shard.shard_batch(p, b, r, G)
            out, ol, ctr = oracle.process_batch(oracle.make_sas(sp), len(sp.spi), sb)
            for j, i in enumerate(idx):
                L = int(ol[j])
                assert L == int(ref_len[i])
                assert out[sb.out_off[j]:sb.out_off[j] + L].tobytes() == \
                    ref_out[b.out_off[i]:b.out_off[i] + L].tobytes()
                seen[i] = True
            for k, v in ctr.as_dict().items():
                tot[k] += v
        valid_sa = b.sa_idx < n_sa
        assert seen[valid_sa].all() and not seen[~valid_sa].any()
        # packets with an invalid SA belong to no shard: the rest matches
        assert tot["pkts_ok"] == ref_ctr.pkts_ok
        assert tot["bytes_out"] == ref_ctr.bytes_out


class _GlooCtx:
    """bench.Ctx's reduction surface on a gloo process group (CPU)."""

    def max_ms(self, ms):
        return shard.max_over_ranks(ms)

    def sum_all(self, d):
        return shard.reduce_counters(d)


def _bench_rates_worker(rank, world, port, out_q):
    import sys
    import torch.distributed as dist
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    # each rank: its own SA shard and batch (weak scaling), a different elapsed time
    p, b = shard.rank_workload(2, 2000, 64 if rank == 0 else "imix", 64, rank, world)
    res = {"b": b, "tot_ms": 10.0 + rank}
    r = bench.rates(_GlooCtx(), res, steps=5)
    out_q.put((rank, r, float(np.asarray(b.frame_len, np.float64).sum()), int(b.in_len.astype(np.int64).sum())))
    dist.barrier()
    dist.destroy_process_group()


def test_bench_rates_whole_job_over_ranks():
    """bench.rates over 2 gloo ranks: value = all ranks' frame bits x steps /
    the MAX elapsed time over ranks (the contract's whole-job aggregate), the
    same on every rank; ESP-payload Gbps from the datagram bytes."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bench_rates_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
    frames = sum(x[2] for x in res)
    payload = sum(x[3] for x in res)
    t = 11.0e-3                                         # max over ranks
    for _, r, _, _ in res:
        assert abs(r["gbps"] - 8 * frames * 5 / t / 1e9) < 1e-9
        assert abs(r["esp_payload_gbps"] - 8 * payload * 5 / t / 1e9) < 1e-9
        assert abs(r["mpps"] - 4000 * 5 / t / 1e6) < 1e-9
        assert abs(r["ms_per_step"] - 11.0 / 5) < 1e-12
