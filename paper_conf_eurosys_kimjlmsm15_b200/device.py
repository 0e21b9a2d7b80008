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
