#!/usr/bin/env python
"""Fixed cost of one ring launch (GPU): event-timed nba_ipsec_ring_run_batches(K)
for several K on the bench's 64-B ring (R device copies, L2-cold), fitted as
T(K) = a + b K; plus the per-batch device timestamps of one K = 20 run (kernel
start -> batch ends).

    python tools/ring_startup.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec, shard  # noqa: E402

p, b = shard.rank_workload(2, 65536, 64, 1024, 0, 1)
t = nba_ipsec.SATable(p, max_batch=65536)
d0 = device.to_device(b, "cuda")
R = device.ring_slot_count(b.in_len, b.n, torch.cuda.get_device_properties(0).L2_cache_size)
dbs = [d0] + [device.clone(d0) for _ in range(R - 1)]
ring = t.ring([(*d.args(), b.n) for d in dbs])
ring.run_batches(4 * R)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
res = {}
for K in (1, 2, 5, 10, 20, 50, 200):
    ms = []
    for _ in range(5):
        torch.cuda.synchronize()
        e0.record()
        ring.run_batches(K)
        e1.record()
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    res[K] = float(np.median(ms)) * 1e3
Ks = np.array(sorted(res))
T = np.array([res[k] for k in Ks])
bfit, afit = np.polyfit(Ks, T, 1)
ts = torch.zeros(21, dtype=torch.int64, device="cuda")
ring.set_timestamps(ts)
ring.run_batches(20)
torch.cuda.synchronize()
v = ts.cpu().numpy().astype(np.int64)
print(json.dumps({"lib": os.environ.get("NBA_IPSEC_LIB", "default"), "us_by_K": {int(k): round(res[k], 2) for k in Ks}, "fit_a_us": round(float(afit), 2),
                  "fit_b_us": round(float(bfit), 3),
                  "ts_first_batch_us": round(float(v[1] - v[0]) / 1e3, 2),
                  "ts_batches_us": [round(float(x) / 1e3, 2) for x in np.diff(v)[1:6]]}), flush=True)
