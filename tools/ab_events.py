"""A/B: step time with and without per-kernel profiling events (PDL overlap)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec
for cfg in (2, 3, 4):
    c = gen.CONFIGS[cfg]
    p = gen.make_sas(c["n_sa"], cfg_id=cfg)
    b = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=cfg)
    t = nba_ipsec.SATable(p, max_batch=c["n"])
    db = device.to_device(b, "cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for prof in (False, True, False):
        t.profile_enable(prof)
        for _ in range(20): t.process(*db.args(), n=b.n)
        torch.cuda.synchronize()
        for flushing in (True, False):
            tot = 0.0
            for _ in range(100):
                if flushing: flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(); t.process(*db.args(), n=b.n); e1.record()
                torch.cuda.synchronize()
                tot += e0.elapsed_time(e1)
            print(f"cfg {cfg} profiling={prof} l2flush={flushing}: {tot/100*1000:.1f} us/step")
    t.close()
