"""A small batch ring (both persistent forms) for compute-sanitizer runs:
    compute-sanitizer --tool racecheck python tools/ring_sanitize.py [pipelined|persistent]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

form = sys.argv[1] if len(sys.argv) > 1 else "pipelined"
n, n_sa = 3000, 16
p = gen.make_sas(n_sa, cfg_id=7)
bs = [gen.make_batch(n, sz, n_sa, cfg_id=7, batch=k) for k, sz in enumerate((64, "imix"))]
sas = oracle.make_sas(p)
with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
    ds = [device.to_device(b, "cuda") for b in bs]
    ring = t.ring([(*d.args(), n) for d in ds])
    if form == "persistent":
        ring.set_form(ring.PERSISTENT)
    ring.run(2)
    torch.cuda.synchronize()
    for b in bs:
        oracle.process_batch(sas, n_sa, b)
    ok = True
    for d, b in zip(ds, bs):
        o_out, o_len, _ = oracle.process_batch(sas, n_sa, b)
        g_out, g_len = device.fetch(d)
        ok &= bool(np.array_equal(g_len, o_len) and np.array_equal(g_out, o_out))
    print(form, "ring == oracle:", ok, "form", ring.form)
    ring.close()
