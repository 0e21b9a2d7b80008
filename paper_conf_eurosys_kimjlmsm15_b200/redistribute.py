"""Single-ingress redistribution: when all traffic
enters at one GPU, each packet must reach the GPU that owns its SA (SA-hash
shard: owner = s mod world) before the ESP path runs there.

  1. nba_ipsec_route_pack (CUDA kernels, libnba_ipsec.so) sorts the ingress
     batch by owner -- stable -- into destination-major send arrays;
  2. exchange() moves them with one all-to-all per array (NCCL over NVLink on
     GPUs; any torch.distributed backend works, tests use gloo on CPU);
  3. each owner runs nba_ipsec_process_batch on what it received (local SA
     indices, packets back to back).

Without the collective: nba_ipsec_route_dispatch routes AND writes every
packet straight into its owner's receive buffers (PeerRx) -- on this GPU or a
peer GPU's memory mapped over NVLink (CUDA IPC: torch shares CUDA tensors
between processes) -- in one pass; see dispatch() below.

This module is plumbing only (sizes, splits, offsets); the routing and packing
arithmetic is in the kernels.
"""
from __future__ import annotations

import dataclasses

import torch
import torch.distributed as dist


@dataclasses.dataclass
class Packed:
    """One rank's destination-major send arrays (output of route_pack)."""
    buf: torch.Tensor        # uint8 [>= total bytes]
    length: torch.Tensor     # int16 [>= total packets] (uint16 values)
    sa: torch.Tensor         # int32 [>= total packets] local SA indices
    counts: list             # packets per destination (world entries)
    nbytes: list             # bytes per destination


@dataclasses.dataclass
class Received:
    """What a rank received: a packed batch for its own SA table."""
    n: int
    in_buf: torch.Tensor     # uint8
    in_off: torch.Tensor     # int32 (uint32 values)
    in_len: torch.Tensor     # int16 (uint16 values)
    sa_idx: torch.Tensor     # int32 local SA indices


def pack(db, n: int, n_sa_total: int, world: int, stream=None, sa_map=None) -> Packed:
    """Route and pack a device batch (gen/device.DeviceBatch with GLOBAL SA
    indices) on the GPU with nba_ipsec_route_pack, or with
    nba_ipsec_route_pack_map when `sa_map` (device uint32 tensor, owner << 24 |
    local, e.g. from the adaptive split, alb.py) is given."""
    from . import nba_ipsec
    dev = db.in_buf.device
    ws = torch.empty(nba_ipsec.route_workspace_bytes(max(n, 1), world), dtype=torch.uint8, device=dev)
    send_buf = torch.empty(max(int(db.in_buf.numel()), 1), dtype=torch.uint8, device=dev)
    send_len = torch.empty(max(n, 1), dtype=torch.int16, device=dev)
    send_sa = torch.empty(max(n, 1), dtype=torch.int32, device=dev)
    dc = torch.zeros(world + 1, dtype=torch.int64, device=dev)
    dbytes = torch.zeros(world + 1, dtype=torch.int64, device=dev)
    if sa_map is None:
        nba_ipsec.route_pack(db.in_buf, db.in_off, db.in_len, db.sa_idx, n, n_sa_total, world, ws,
                             send_buf, send_len, send_sa, dc, dbytes, stream=stream)
    else:
        nba_ipsec.route_pack_map(db.in_buf, db.in_off, db.in_len, db.sa_idx, n, n_sa_total, sa_map,
                                 world, ws, send_buf, send_len, send_sa, dc, dbytes, stream=stream)
    c = dc.cpu().tolist()
    b = dbytes.cpu().tolist()
    return Packed(buf=send_buf, length=send_len, sa=send_sa, counts=c[:world], nbytes=b[:world])


def exchange(p: Packed, group=None) -> Received:
    """All-to-all of the packed arrays; returns this rank's received batch.
    Every rank calls it (ranks without ingress traffic pass empty arrays)."""
    world = dist.get_world_size(group)
    dev = p.buf.device
    sizes = torch.tensor([p.counts, p.nbytes], dtype=torch.int64).t().contiguous().to(dev)
    got = torch.empty_like(sizes)
    dist.all_to_all_single(got, sizes, group=group)
    got = got.cpu()
    r_cnt = got[:, 0].tolist()
    r_byt = got[:, 1].tolist()
    n_in, b_in = sum(p.counts), sum(p.nbytes)
    n_out, b_out = sum(r_cnt), sum(r_byt)
    # lengths travel as bytes (16-bit integers are not an NCCL type)
    len_bytes = torch.empty(max(2 * n_out, 1), dtype=torch.uint8, device=dev)
    dist.all_to_all_single(len_bytes[:2 * n_out], p.length[:n_in].view(torch.uint8)[:2 * n_in],
                           [2 * c for c in r_cnt], [2 * c for c in p.counts], group=group)
    sa = torch.empty(max(n_out, 1), dtype=torch.int32, device=dev)
    dist.all_to_all_single(sa[:n_out], p.sa[:n_in], r_cnt, p.counts, group=group)
    buf = torch.empty(max(b_out, 1) + 16, dtype=torch.uint8, device=dev)
    dist.all_to_all_single(buf[:b_out], p.buf[:b_in], r_byt, p.nbytes, group=group)
    length = len_bytes[:2 * n_out].view(torch.int16) if n_out else torch.zeros(1, dtype=torch.int16,
                                                                                 device=dev)
    lens = length[:n_out].to(torch.int64) & 0xFFFF
    off = torch.zeros(max(n_out, 1), dtype=torch.int64, device=dev)
    if n_out > 1:
        off[1:n_out] = torch.cumsum(lens[:-1], 0)
    return Received(n=n_out, in_buf=buf, in_off=off.to(torch.int32), in_len=length, sa_idx=sa)


def local_views(p: Packed, d: int, out_pad: int = 64):
    """One destination's region of the packed arrays as a batch for that
    owner's table on THIS device (the one-process stand-in for the exchange,
    used by the adaptive split, alb.py): (n, in_off, in_len, sa_idx, out_off,
    out_len, out_buf), offsets into p.buf / a fresh output pool."""
    dev = p.buf.device
    c0, b0 = sum(p.counts[:d]), sum(p.nbytes[:d])
    n = p.counts[d]
    lens = p.length[c0:c0 + n].to(torch.int64) & 0xFFFF
    in_off = torch.full((max(n, 1),), b0, dtype=torch.int64, device=dev)
    out_off = torch.zeros(max(n, 1), dtype=torch.int64, device=dev)
    if n > 1:
        in_off[1:n] += torch.cumsum(lens[:-1], 0)
        out_off[1:n] = torch.cumsum(lens[:-1] + out_pad, 0)
    pool = int(p.nbytes[d]) + out_pad * n + 16
    out_buf = torch.empty(pool, dtype=torch.uint8, device=dev)
    out_len = torch.empty(max(n, 1), dtype=torch.int16, device=dev)
    return (n, in_off.to(torch.int32), p.length[c0:], p.sa[c0:], out_off.to(torch.int32), out_len,
            out_buf)


# ---- single-ingress dispatch over peer memory (no send buffer, no NCCL) --------

@dataclasses.dataclass
class PeerRx:
    """One owner's receive buffers (device tensors on the owner's GPU; another
    process may hold them through CUDA IPC)."""
    buf: torch.Tensor        # uint8 [cap_bytes]
    off: torch.Tensor        # int32 [cap_pkts]
    length: torch.Tensor     # int16 [cap_pkts]
    sa: torch.Tensor         # int32 [cap_pkts]
    count: torch.Tensor      # int64 [2]: packets, bytes


def alloc_rx(cap_pkts: int, cap_bytes: int, device) -> PeerRx:
    return PeerRx(buf=torch.empty(max(cap_bytes, 16), dtype=torch.uint8, device=device),
                  off=torch.empty(max(cap_pkts, 1), dtype=torch.int32, device=device),
                  length=torch.empty(max(cap_pkts, 1), dtype=torch.int16, device=device),
                  sa=torch.empty(max(cap_pkts, 1), dtype=torch.int32, device=device),
                  count=torch.zeros(2, dtype=torch.int64, device=device))


def rx_table(rxs, device) -> torch.Tensor:
    """Device array of nba_ipsec_peer_rx descriptors (5 pointers each), with the
    pointers as seen by THIS process (own or IPC-mapped tensors)."""
    ptrs = [[r.buf.data_ptr(), r.off.data_ptr(), r.length.data_ptr(), r.sa.data_ptr(),
             r.count.data_ptr()] for r in rxs]
    return torch.tensor(ptrs, dtype=torch.int64).view(-1).to(device)


def dispatch(db, n: int, n_sa_total: int, world: int, table: torch.Tensor, cap_pkts: int,
             cap_bytes: int, sa_map=None, stream=None):
    """Route a device batch with GLOBAL SA indices and write each packet into its
    owner's receive buffers (nba_ipsec_route_dispatch).  Returns the per-owner
    (packets, bytes) counts (read back; synchronises)."""
    from . import nba_ipsec
    dev = db.in_buf.device
    ws = torch.empty(nba_ipsec.route_workspace_bytes(max(n, 1), world), dtype=torch.uint8, device=dev)
    dc = torch.zeros(world + 1, dtype=torch.int64, device=dev)
    dbytes = torch.zeros(world + 1, dtype=torch.int64, device=dev)
    nba_ipsec.route_dispatch(db.in_buf, db.in_off, db.in_len, db.sa_idx, n, n_sa_total, sa_map,
                             world, ws, table, cap_pkts, cap_bytes, dc, dbytes, stream=stream)
    return dc.cpu().tolist()[:world], dbytes.cpu().tolist()[:world]


def received_batch(rx: PeerRx):
    """(n, in_buf, in_off, in_len, sa_idx) of what the dispatch wrote into rx, as
    process_batch arguments (device tensors; n read back)."""
    n = int(rx.count[0].item())
    return n, rx.buf, rx.off, rx.length, rx.sa
