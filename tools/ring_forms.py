#!/usr/bin/env python
"""The outbound ring's persistent forms side by side (GPU), bench protocol:
R device copies of one full-size batch (65,536 packets, 1024 SAs), >= 2R
warm-up batches, then K = 200 batches in ONE nba_ipsec_ring_run_batches call
between one CUDA event pair (a sleep kernel ahead of the start event), per
form (nba_ipsec_ring_set_form), two passes interleaved.

    FORMS=pipelined,roles RING_K=200 python tools/ring_forms.py [sizes...]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec, shard  # noqa: E402

K = 200
sizes = [x if x == "imix" else int(x) for x in sys.argv[1:]] or [64, 1514, "imix"]
ALL = {"pipelined": nba_ipsec.Ring.PIPELINED, "free": nba_ipsec.Ring.FREE, "roles": nba_ipsec.Ring.ROLES,
       "persistent": nba_ipsec.Ring.PERSISTENT}
forms = {f: ALL[f] for f in os.environ.get("FORMS", "pipelined,roles").split(",")}
K = int(os.environ.get("RING_K", K))
res = {f: {} for f in forms}
for size in sizes:
    cfg = {64: 2, 1514: 3, "imix": 4}.get(size, 5)
    p, b = shard.rank_workload(cfg, 65536, size, 1024, 0, 1)
    t = nba_ipsec.SATable(p, max_batch=65536)
    d0 = device.to_device(b, "cuda")
    R = device.ring_slot_count(b.in_len, b.n, torch.cuda.get_device_properties(0).L2_cache_size)
    dbs = [d0] + [device.clone(d0) for _ in range(R - 1)]
    ring = t.ring([(*d.args(), b.n) for d in dbs])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for rep in range(2):
        for name, f in forms.items():
            ring.set_form(f)
            ring.run_batches(2 * R)
            torch.cuda.synchronize()
            torch.cuda._sleep(200000)
            e0.record()
            ring.run_batches(K)
            e1.record()
            torch.cuda.synchronize()
            res[name].setdefault(str(size), []).append(round(e0.elapsed_time(e1) * 1e3 / K, 2))
    ring.close()
    t.close()
print(json.dumps(res), flush=True)

if os.environ.get("FREE_TRACE"):
    # trace variant (NBA_RING_TRACE=1 via NBA_IPSEC_LIB): per batch (median over
    # CTAs, relative to the batch's earliest side start): 0 side start, 1 prologue
    # + placement done, 2 published, 3 latest lane take, 4 latest lane finish,
    # 6 longest lane wait
    import numpy as np
    out = {}
    for size in sizes:
        cfg = {64: 2, 1514: 3, "imix": 4}.get(size, 5)
        p, b = shard.rank_workload(cfg, 65536, size, 1024, 0, 1)
        t = nba_ipsec.SATable(p, max_batch=65536)
        d0 = device.to_device(b, "cuda")
        R = device.ring_slot_count(b.in_len, b.n, torch.cuda.get_device_properties(0).L2_cache_size)
        dbs = [d0] + [device.clone(d0) for _ in range(R - 1)]
        ring = t.ring([(*d.args(), b.n) for d in dbs])
        ring.set_form(nba_ipsec.Ring.FREE)
        ring.run_batches(2 * R)
        torch.cuda.synchronize()
        nb, G = 12, 148
        ts = torch.zeros(nb * G * 16, dtype=torch.int64, device="cuda")
        ring.set_timestamps(ts)
        ring.run_batches(nb)
        torch.cuda.synchronize()
        v = ts.cpu().numpy().reshape(nb, G, 16).astype(np.int64)
        t0 = v[:, :, 0].min(axis=1, keepdims=True)
        rel = (v - t0[:, :, None]) / 1e3
        rel[:, :, 6] = v[:, :, 6] / 1e3
        starts = v[:, :, 0].min(axis=1)
        out[str(size)] = {"batch_period_us": [round(float(x) / 1e3, 1) for x in np.diff(starts)],
                          **{n: round(float(np.median(rel[2:-1, :, k])), 2) for k, n in
                             [(1, "prologue_placed"), (2, "published"), (3, "last_take"),
                              (4, "last_finish"), (6, "longest_wait")]}}
        ring.close()
        t.close()
    print(json.dumps(out), flush=True)
