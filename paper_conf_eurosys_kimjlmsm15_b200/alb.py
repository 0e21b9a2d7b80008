"""Adaptive split of the SAs across devices -- plumbing.

PAPER.md:351-365 (§3.4): NBA's load balancer hill-climbs the offloading
fraction w by delta on the moving-average throughput.  On a B200 box the split
that matters is which GPU owns which SAs (S§8(e): with single ingress a GPU
processes exactly the packets of its SAs, and an SA's counter lives on its
owner).  The controller and the SA assignment are the library's host code
(``nba_ipsec_alb_*``, csrc/alb.cpp); this module only

  * arranges one controller per internal node of the binary device tree
    (reading L6) and feeds each the throughput of its subtree,
  * turns the node steps into an owner map (``nba_ipsec_alb_assign``), and
  * hands the sequence counters of SAs that change owner to the new owner
    (reading L7): a MAX all-reduce of the old owners' counters over the
    process group (one small collective per ownership change, NCCL on GPUs),
    or, for several tables in one process, a read/write through the C ABI.
"""
from __future__ import annotations

import numpy as np

from . import nba_ipsec


def internal_nodes(n_dev: int) -> list[tuple[int, int, int]]:
    """(heap id, lo, hi) of every internal node of the device tree (L6)."""
    out = []

    def rec(node, lo, hi):
        if hi - lo < 2:
            return
        out.append((node, lo, hi))
        mid = lo + (hi - lo) // 2
        rec(2 * node + 1, lo, mid)
        rec(2 * node + 2, mid, hi)

    rec(0, 0, n_dev)
    return out


class Balancer:
    """One nba_ipsec_alb controller per internal node of the device tree."""

    def __init__(self, n_sa: int, n_dev: int, **params):
        if not 1 <= n_dev <= nba_ipsec.ALB_MAX_DEV:
            raise ValueError("n_dev must be 1..8")
        self.n_sa, self.n_dev = int(n_sa), int(n_dev)
        self.nodes = internal_nodes(self.n_dev)
        self.ctl = {nid: nba_ipsec.Alb(**params) for nid, _, _ in self.nodes}
        self.steps = int(nba_ipsec.alb_default_params().steps if params.get("steps") is None
                         else params["steps"])
        self.node_step = np.zeros(nba_ipsec.ALB_TREE_NODES, np.uint32)
        for nid, c in self.ctl.items():
            self.node_step[nid] = c.state()[0]

    def assignment(self):
        """(owner[n_sa], sa_map[n_sa]) for the current node steps."""
        return nba_ipsec.alb_assign(self.n_sa, self.n_dev, self.node_step, self.steps)

    def observe(self, t_ns: int, dev_dt_ns, dev_pkts) -> bool:
        """One step's sample: per device its busy time (ns) and packets out.
        A node's sample is its subtree's packets over its slowest device's
        time.  Returns True if any node changed its step."""
        changed = False
        for nid, lo, hi in self.nodes:
            dt = int(max(int(x) for x in dev_dt_ns[lo:hi]))
            p = int(sum(int(x) for x in dev_pkts[lo:hi]))
            k = self.ctl[nid].observe(int(t_ns), dt, p)
            if k != self.node_step[nid]:
                self.node_step[nid] = k
                changed = True
        return changed


def handover_tables(tables, old_owner, new_owner, stream=None):
    """Several SA tables in one process (each holding every SA): the counter of
    every SA is taken from its old owner's table and written to its new
    owner's (reading L7).  Only tables that gain SAs are written."""
    old_owner = np.asarray(old_owner)
    new_owner = np.asarray(new_owner)
    seqs = [t.sa_seq(stream) for t in tables]
    live = np.zeros(len(old_owner), np.uint32)
    for d, s in enumerate(seqs):
        live[old_owner == d] = s[old_owner == d]
    for d, t in enumerate(tables):
        gain = (new_owner == d) & (old_owner != d)
        if gain.any():
            s = seqs[d].copy()
            s[gain] = live[gain]
            t.write_sa_seq(s, stream)


def handover_dist(table, old_owner, rank: int, group=None, device=None, stream=None):
    """One table per rank: MAX all-reduce of the counters each rank owned under
    `old_owner` (zero elsewhere); every rank then holds the live counter of
    every SA and writes it to its table (the old owner's value is the only
    nonzero contribution, and a counter never decreases)."""
    import torch
    import torch.distributed as dist
    s = table.sa_seq(stream).astype(np.int64)
    s[np.asarray(old_owner) != rank] = 0
    t = torch.from_numpy(s).to(device) if device is not None else torch.from_numpy(s)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    table.write_sa_seq(t.cpu().numpy().astype(np.uint32), stream)
