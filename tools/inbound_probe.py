"""Inbound back-to-back vs isolated: which factor costs the difference?
64 B config.  (a) rotation over R ESP batches, windows reset only at wrap (the
bench protocol); (b) the same with a window reset before every batch; (c) one
ESP batch re-used every step with a reset before each (no rotation); (d) as
(c) with an L2 flush + per-batch events (the isolated protocol)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

p = gen.make_sas(1024, cfg_id=2)
b = gen.make_batch(65536, 64, 1024, cfg_id=2)
t_out = nba_ipsec.SATable(p, max_batch=b.n)
db = device.to_device(b, "cuda")
R = int(sys.argv[1]) if len(sys.argv) > 1 else 9
esp = []
for _ in range(R):
    ob, ol = torch.empty_like(db.out_buf), torch.zeros_like(db.out_len)
    t_out.process(db.in_buf, db.in_off, db.in_len, db.sa_idx, ob, db.out_off, ol, n=b.n)
    esp.append((ob, ol, torch.empty_like(db.out_buf), torch.zeros_like(db.out_len)))
torch.cuda.synchronize()
t = nba_ipsec.SATable(p, max_batch=b.n)
t.enable_inbound()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def run(k, reset_every, rot):
    j = k % R if rot else 0
    if reset_every or j == 0:
        t.reset_inbound()
    ob, ol, inner, il = esp[j]
    t.process_inbound(ob, db.out_off, ol, db.sa_idx, inner, db.out_off, il, n=b.n)


K = 200
for name, reset_every, rot in (("a rotate, reset at wrap", False, True),
                               ("b rotate, reset every batch", True, True),
                               ("c one batch, reset every batch", True, False)):
    for k in range(2 * R):
        run(k, reset_every, rot)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for k in range(K):
        run(k, reset_every, rot)
    e1.record()
    torch.cuda.synchronize()
    print(f"{name}: {e0.elapsed_time(e1) / K * 1e3:.1f} us/step (R={R})", flush=True)
tot = 0.0
for k in range(50):
    flush.zero_()
    t.reset_inbound()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    ob, ol, inner, il = esp[0]
    t.process_inbound(ob, db.out_off, ol, db.sa_idx, inner, db.out_off, il, n=b.n)
    e1.record()
    torch.cuda.synchronize()
    tot += e0.elapsed_time(e1)
print(f"d isolated (flush, events per batch): {tot / 50 * 1e3:.1f} us/step")
print("launches per batch:", t.inbound_launches_per_batch(), "counters:", t.in_counters())
