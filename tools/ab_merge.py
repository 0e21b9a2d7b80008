"""A/B: merged (prologue inside the fused kernel, 1 launch) vs the two-kernel
fused path, same protocol as bench.py (L2 flush before each step, per-step
CUDA events, host runs ahead)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timed(t, db, n, steps=200):
    for _ in range(30):
        flush.zero_()
        t.process(*db.args(), n=n)
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(steps)]
    for k in range(steps):
        flush.zero_()
        ev[k][0].record()
        t.process(*db.args(), n=n)
        ev[k][1].record()
    torch.cuda.synchronize()
    return sum(a.elapsed_time(b) for a, b in ev) / steps * 1000


for cfg in ([int(x) for x in sys.argv[1:]] or (2, 3, 4)) if __name__ == "__main__" else ():
    c = gen.CONFIGS[cfg]
    p = gen.make_sas(c["n_sa"], cfg_id=cfg)
    b = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=cfg)
    db = device.to_device(b, "cuda")
    tm = nba_ipsec.SATable(p, max_batch=c["n"])
    os.environ["NBA_IPSEC_NO_MERGE"] = "1"
    t2 = nba_ipsec.SATable(p, max_batch=c["n"])
    del os.environ["NBA_IPSEC_NO_MERGE"]
    for rep in range(2):
        a = timed(tm, db, b.n)
        bb = timed(t2, db, b.n)
        print(f"cfg {cfg}: merged {a:.1f} us/step ({tm.launches_per_batch()} launch), "
              f"two-kernel {bb:.1f} us/step ({t2.launches_per_batch()} launches)")
    tm.close()
    t2.close()
