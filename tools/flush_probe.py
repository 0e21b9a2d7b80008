"""Step time of the fused path with and without the bench's L2 flush between
steps (the flush kernel also changes the SM's L1/shared-memory carve-out)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

for cfg in (2, 3):
    c = gen.CONFIGS[cfg]
    p = gen.make_sas(c["n_sa"], cfg_id=cfg)
    b = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=cfg)
    db = device.to_device(b, "cuda")
    t = nba_ipsec.SATable(p, max_batch=c["n"])
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for mode in ("torch-fill", "none", "memset"):
        for _ in range(30):
            t.process(*db.args(), n=b.n)
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(200)]
        for k in range(200):
            if mode == "torch-fill":
                flush.zero_()
            elif mode == "memset":
                torch.cuda.memset_async = None
                flush.fill_(1)
            ev[k][0].record()
            t.process(*db.args(), n=b.n)
            ev[k][1].record()
        torch.cuda.synchronize()
        ms = sum(a.elapsed_time(e) for a, e in ev) / 200
        print(f"cfg {cfg} flush={mode}: {ms * 1000:.1f} us/step")
    t.close()
