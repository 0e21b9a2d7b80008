"""Run a few ESP inbound batches of a bench config through the C ABI (for ncu
captures): the library's own outbound output is decapsulated, windows reset
between batches.  --ring: through an inbound ring of 4 slots (one launch of
`batches` batches; the form the library picks, or NBA_IPSEC_RING_IN_PIPE)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=2)
ap.add_argument("--batches", type=int, default=3)
ap.add_argument("--ring", action="store_true")
a = ap.parse_args()
c = gen.CONFIGS[a.config]
p = gen.make_sas(c["n_sa"], cfg_id=a.config)
b = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=a.config)
t_out = nba_ipsec.SATable(p, max_batch=c["n"])
db = device.to_device(b, "cuda")
t_out.process(*db.args(), n=b.n)
t = nba_ipsec.SATable(p, max_batch=c["n"])
t.enable_inbound()
inner = torch.empty_like(db.out_buf)
il = torch.zeros_like(db.out_len)
if a.ring:
    slots = [(db.out_buf, db.out_off, db.out_len, db.sa_idx, torch.empty_like(db.out_buf), db.out_off,
              torch.zeros_like(db.out_len), None, b.n) for _ in range(4)]
    ring = t.ring_inbound(slots)
    t.reset_inbound()
    ring.run_batches(a.batches)
    torch.cuda.synchronize()
    print("form", ring.form)
    ring.close()
else:
    for _ in range(a.batches):
        t.reset_inbound()
        t.process_inbound(db.out_buf, db.out_off, db.out_len, db.sa_idx, inner, db.out_off, il, n=b.n)
torch.cuda.synchronize()
print("ok", t.in_counters())
