"""Device-memory plumbing for batches (torch tensors as byte buffers).

Moves a gen.Batch into CUDA tensors with the C ABI's element types
(u8 / u32 / u16 reinterpreted as torch uint8 / int32 / int16) and back.
No ESP arithmetic here.
"""
from __future__ import annotations

import dataclasses

import numpy as np
import torch


@dataclasses.dataclass
class DeviceBatch:
    n: int
    in_buf: torch.Tensor
    in_off: torch.Tensor
    in_len: torch.Tensor
    sa_idx: torch.Tensor
    out_buf: torch.Tensor
    out_off: torch.Tensor
    out_len: torch.Tensor

    def args(self):
        return (self.in_buf, self.in_off, self.in_len, self.sa_idx, self.out_buf, self.out_off,
                self.out_len)


def _t(a: np.ndarray, dt, device):
    return torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(device)


def to_device(b, device="cuda", out_fill: int | None = 0) -> DeviceBatch:
    n = int(b.n)
    out = (torch.zeros if out_fill == 0 else torch.empty)(max(b.out_pool_bytes, 1),
                                                           dtype=torch.uint8, device=device)
    if out_fill not in (None, 0):
        out.fill_(out_fill)
    return DeviceBatch(
        n=n,
        in_buf=_t(b.in_buf, np.uint8, device),
        in_off=_t(b.in_off.astype(np.uint32), np.int32, device),
        in_len=_t(b.in_len.astype(np.uint16), np.int16, device),
        sa_idx=_t(b.sa_idx.astype(np.uint32), np.int32, device),
        out_buf=out,
        out_off=_t(b.out_off.astype(np.uint32), np.int32, device),
        out_len=torch.zeros(max(n, 1), dtype=torch.int16, device=device),
    )


def fetch(db: DeviceBatch):
    torch.cuda.synchronize(db.out_buf.device)
    out = db.out_buf.cpu().numpy()
    ol = db.out_len[:db.n].cpu().numpy().view(np.uint16)
    return out, ol


def ring_slot_count(in_len: np.ndarray, n: int, l2_bytes: int) -> int:
    """Device copies of a batch the benchmark rotates over so that one rotation
    touches more than 2x the L2 (every batch starts L2-cold): bytes touched per
    batch ~ the datagrams plus, per packet, the 128-byte lines of its input and
    output slots and its metadata.  Shared by bench.py and the tests that
    check the bench's exact ring."""
    touched = int(np.asarray(in_len, np.int64).sum()) + int(n) * (128 + 53 + 128 + 14)
    return max(2, -(-2 * int(l2_bytes) // touched))


def clone(d: DeviceBatch) -> DeviceBatch:
    """A second device copy of a batch (fresh output pool / lengths)."""
    return DeviceBatch(n=d.n, in_buf=d.in_buf.clone(), in_off=d.in_off.clone(),
                       in_len=d.in_len.clone(), sa_idx=d.sa_idx.clone(),
                       out_buf=torch.zeros_like(d.out_buf), out_off=d.out_off.clone(),
                       out_len=torch.zeros_like(d.out_len))
