"""Multi-GPU plumbing: SA-hash sharding and the end-of-run reductions.

SURVEY.md §8(e) / DESIGN.md §6: packets are independent given their SA's
sequence counter, so GPU g owns the SAs with s mod G == g (and their counters)
and never exchanges packets with other GPUs -- the analogue of NBA's
replicated, shared-nothing worker pipelines.  The only
collectives are end-of-run: a SUM all-reduce of the int64 counters and a MAX
all-reduce of the elapsed time (NCCL over NVLink on GPUs, gloo on CPU).
"""
from __future__ import annotations

import numpy as np

from . import gen

COUNTER_KEYS = ("pkts_ok", "pkts_dropped", "bytes_in", "bytes_out", "batches")


def owner(s, world: int):
    """GPU (rank) that owns global SA s."""
    return np.asarray(s) % world


def shard_params(p: gen.SAParams, rank: int, world: int) -> gen.SAParams:
    """The SAs rank owns, renumbered densely (local index = s // world)."""
    idx = np.arange(rank, len(p.spi), world)
    return gen.SAParams(*(np.array(getattr(p, f)[idx]) for f in
                          ("spi", "tunnel_src", "tunnel_dst", "aes_key", "ctr_nonce",
                           "hmac_key", "seq")))


def shard_batch(p: gen.SAParams, b: gen.Batch, rank: int, world: int):
    """Packets of batch b that rank owns, in their original order (per-SA order
    is what fixes sequence numbers, so order within a shard is preserved).
    Returns (shard params, shard batch with local SA indices, original indices)."""
    n_sa = len(p.spi)
    sel = (b.sa_idx < n_sa) & (owner(b.sa_idx, world) == rank)
    idx = np.nonzero(sel)[0]
    sb = gen.Batch(n=int(idx.size), in_buf=b.in_buf, in_off=b.in_off[idx], in_len=b.in_len[idx],
                   sa_idx=(b.sa_idx[idx] // world).astype(np.uint32), out_off=b.out_off[idx],
                   out_pool_bytes=b.out_pool_bytes, frame_len=b.frame_len[idx])
    return shard_params(p, rank, world), sb, idx


def rank_workload(cfg_id: int, n: int, size, n_sa_total: int, rank: int, world: int,
                  batch: int = 0, **kw):
    """Weak-scaling workload of one rank: its own SA shard (n_sa_total/world SAs,
    global ids rank + world*j) and its own batch of n packets over them."""
    n_local = len(range(rank, n_sa_total, world))
    p = gen.make_sas(n_local, cfg_id=cfg_id, rank=rank, world=world)
    b = gen.make_batch(n, size, n_local, cfg_id=cfg_id, rank=rank, batch=batch, **kw)
    return p, b


def reduce_counters(c: dict, device=None) -> dict:
    """SUM all-reduce of the device counters over the default process group."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([int(c[k]) for k in COUNTER_KEYS], dtype=torch.int64, device=device)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return dict(zip(COUNTER_KEYS, (int(x) for x in t.tolist())))


def max_over_ranks(x: float, device=None) -> float:
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
