"""Run a few batches of a bench config through the C ABI (for ncu captures)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--batches", type=int, default=3)
ap.add_argument("--pipeline", type=int, default=None)
ap.add_argument("--ring", type=int, default=0,
                help="R > 0: run --batches rounds of an R-slot batch ring (device copies)")
a = ap.parse_args()
c = gen.CONFIGS[a.config]
p = gen.make_sas(c["n_sa"], cfg_id=a.config)
b = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=a.config)
t = nba_ipsec.SATable(p, max_batch=c["n"])
if a.pipeline is not None:
    t.set_pipeline(a.pipeline)
db = device.to_device(b, "cuda")
if a.ring:
    dbs = [db] + [device.to_device(b, "cuda") for _ in range(a.ring - 1)]
    ring = t.ring([(*d.args(), b.n) for d in dbs])
    ring.run(a.batches)
else:
    for _ in range(a.batches):
        t.process(*db.args(), n=b.n)
torch.cuda.synchronize()
print("ok", t.counters())
