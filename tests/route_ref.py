"""Plain numpy statement of single-ingress routing (tests only): a stable
partition of the batch by owner = s mod world (s < n_sa_total; others are not
sent), packets back to back per destination, local SA index s / world.  With
an explicit map (the adaptive split): owner = map[s] >> 24 (not sent
if >= world), local index map[s] & 0xFFFFFF."""
import numpy as np
import torch

from paper_conf_eurosys_kimjlmsm15_b200.redistribute import Packed


def route_pack_ref(b, n_sa_total, world, sa_map=None):
    s = b.sa_idx.astype(np.int64)
    ok = s < n_sa_total
    if sa_map is None:
        dest = np.where(ok, s % world, world)
        local = s // world
    else:
        m = np.asarray(sa_map, np.int64)
        e = m[np.where(ok, s, 0)]
        dest = np.where(ok, np.minimum(e >> 24, world), world)
        local = e & 0xFFFFFF
    bufs, lens, sas, counts, nbytes = [], [], [], [], []
    for d in range(world):
        idx = np.nonzero(dest == d)[0]
        counts.append(int(idx.size))
        nbytes.append(int(b.in_len[idx].astype(np.int64).sum()))
        for i in idx:
            bufs.append(b.in_buf[b.in_off[i]:b.in_off[i] + b.in_len[i]])
            lens.append(int(b.in_len[i]))
            sas.append(int(local[i]))
    buf = np.concatenate(bufs) if bufs else np.zeros(0, np.uint8)
    return buf, np.array(lens, np.uint16), np.array(sas, np.uint32), counts, nbytes


def packed_cpu(b, n_sa_total, world, sa_map=None):
    buf, lens, sas, counts, nbytes = route_pack_ref(b, n_sa_total, world, sa_map)
    return Packed(buf=torch.from_numpy(buf.copy()) if buf.size else torch.zeros(1, dtype=torch.uint8),
                  length=torch.from_numpy(lens.view(np.int16).copy()) if lens.size else
                  torch.zeros(1, dtype=torch.int16),
                  sa=torch.from_numpy(sas.view(np.int32).copy()) if sas.size else
                  torch.zeros(1, dtype=torch.int32),
                  counts=counts, nbytes=nbytes)
