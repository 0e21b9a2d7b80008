#!/usr/bin/env python
"""DRAM bytes of the 64-B ring under different output-slot alignments (run
under ncu, one k_fused_ring_pipe launch of 4 batches per layout):

    ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum -k regex:k_fused_ring \\
        python tools/traffic_probe.py {bench,out128,out128in128}

bench       the bench layout: datagrams and output slots at 2048 i + 142
            (= 14 mod 16; the 100-byte ESP packet covers two partial sectors)
out128      output slots at 2048 i + 128 (one partial sector, at the end)
out128in128 datagrams at 2048 i + 128 too (50 bytes in two sectors, 64 read)
If partial-sector writes cost DRAM fills, `out128` reads ~2 MB less per batch."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec, shard  # noqa: E402

mode = sys.argv[1] if len(sys.argv) > 1 else "bench"
p, b = shard.rank_workload(2, 65536, 64, 1024, 0, 1)
if mode in ("out128", "out128in128"):
    b.out_off = (b.out_off - 14).astype(np.uint32)
if mode == "out128in128":
    buf = np.zeros_like(b.in_buf)
    for i in range(b.n):
        o = int(b.in_off[i])
        buf[o - 14:o - 14 + int(b.in_len[i])] = b.in_buf[o:o + int(b.in_len[i])]
    b.in_buf = buf
    b.in_off = (b.in_off - 14).astype(np.uint32)
t = nba_ipsec.SATable(p, max_batch=65536)
dbs = [device.to_device(b, "cuda") for _ in range(4)]
ring = t.ring([(*d.args(), b.n) for d in dbs])
ring.run_batches(4)
torch.cuda.synchronize()
print(mode, "ok", t.counters())
