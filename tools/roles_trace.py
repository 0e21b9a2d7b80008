#!/usr/bin/env python
"""Phase trace of the role-split ring (GPU; needs the NBA_ROLES_TRACE=1 build,
`python tools/ring_ab.py build rtrace=NBA_ROLES_TRACE=1`, loaded through
NBA_IPSEC_LIB): per batch, sequencer 0's phases (consumed wait, A = ranks,
B = per-warp prefix, barrier among sequencers, C = per-SA bases, D = records
out) and when lane CTA 0 started waiting for / received the batch's records;
medians over batches 4..K-2 of each phase's duration and of the batch period.

    NBA_IPSEC_LIB=build/variants/rtrace.so [NBA_IPSEC_ROLES_P=4] python tools/roles_trace.py [sizes...]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec, shard  # noqa: E402

K = 50
out = {}
for size in [x if x == "imix" else int(x) for x in sys.argv[1:]] or [64]:
    cfg = {64: 2, 1514: 3, "imix": 4}.get(size, 5)
    p, b = shard.rank_workload(cfg, 65536, size, 1024, 0, 1)
    t = nba_ipsec.SATable(p, max_batch=65536)
    d0 = device.to_device(b, "cuda")
    R = device.ring_slot_count(b.in_len, b.n, torch.cuda.get_device_properties(0).L2_cache_size)
    dbs = [d0] + [device.clone(d0) for _ in range(R - 1)]
    ring = t.ring([(*d.args(), b.n) for d in dbs])
    ring.set_form(nba_ipsec.Ring.ROLES)
    ring.run_batches(2 * R)
    ts = torch.zeros(K * 9 + 1 + 4 * 4 * 512 * 2, dtype=torch.int64, device="cuda")
    ring.set_timestamps(ts)
    ring.run_batches(K)
    torch.cuda.synchronize()
    v = ts.cpu().numpy().astype(np.int64)
    ends = v[1:K + 1]
    st = v[K + 1:K + 1 + 8 * K].reshape(K, 8)
    lt = v[1 + 9 * K:].reshape(4, 4, 512, 2)
    lanes_tl = {}
    for bb in range(4):
        x = lt[bb].reshape(-1, 2)
        x = x[(x[:, 0] > 0) & (x[:, 1] > 0)]
        if len(x):
            rel0 = (x[:, 0] - v[0]) / 1e3
            dur = (x[:, 1] - x[:, 0]) / 1e3
            lanes_tl[bb] = {"n": int(len(x)), "start_us_p10_50_90": [round(float(np.percentile(rel0, q)), 2) for q in (10, 50, 90)],
                            "dur_us_p10_50_90": [round(float(np.percentile(dur, q)), 2) for q in (10, 50, 90)],
                            "end_us_max": round(float(((x[:, 1] - v[0]) / 1e3).max()), 2)}
    sl = slice(4, K - 1)
    med = lambda a: round(float(np.median(a[sl])) / 1e3, 2)  # noqa: E731
    out[str(size)] = {
        "batch_period_us": med(np.diff(ends, prepend=ends[0])),
        "seq_period_us": med(np.diff(st[:, 5], prepend=st[0, 5])),
        "seq_A_ranks_incl_consumed_wait": med(st[:, 1] - st[:, 0]),
        "seq_B_prefix": med(st[:, 2] - st[:, 1]),
        "seq_barrier": med(st[:, 3] - st[:, 2]),
        "seq_C_bases": med(st[:, 4] - st[:, 3]),
        "seq_D_records": med(st[:, 5] - st[:, 4]),
        "seq_idle_between": med(st[1:, 0] - st[:-1, 5]),
        "lane0_wait_for_records": med(st[:, 7] - st[:, 6]),
        "records_lead_over_lane0_us": med(st[:, 6] - st[:, 5]),
        "first_batch_end_us": round(float(ends[0] - v[0]) / 1e3, 2),
        "lanes_first_batches": lanes_tl,
        # batches 0..2 from the kernel start: sequencer 0's stamps (phase start, A, B,
        # barrier, C, D/published), lane CTA 0's wait start / records seen, batch end
        "start_batches_0_2_us": [[round(float(x - v[0]) / 1e3, 2) for x in list(st[b]) + [ends[b]]]
                                 for b in range(3)],
    }
    ring.close()
    t.close()
print(json.dumps(out), flush=True)
