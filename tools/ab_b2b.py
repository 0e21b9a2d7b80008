"""A/B of library variants under the bench's headline protocol: K batches back
to back on one stream between one CUDA event pair, rotating over device copies
of the batch that touch > 2x L2.

    python tools/ab_b2b.py [lib.so ...]     (GPU; default: the in-tree library)

Each variant runs in a fresh process through NBA_IPSEC_LIB, twice, interleaved."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

TIMER = r'''
import os, sys
sys.path.insert(0, %r)
import numpy as np, torch
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec
L2 = torch.cuda.get_device_properties(0).L2_cache_size
for cfg, size in [c for c in ((2, 64), (3, 1514), (4, "imix")) if str(c[0]) in os.environ.get("AB_CFGS", "234")]:
    p = gen.make_sas(1024, cfg_id=cfg)
    b = gen.make_batch(65536, size, 1024, cfg_id=cfg)
    db = device.to_device(b, "cuda")
    touched = int(b.in_len.astype(np.int64).sum()) + b.n * 451
    R = max(2, -(-2 * L2 // touched))
    dbs = [db] + [device.DeviceBatch(n=db.n, in_buf=db.in_buf.clone(), in_off=db.in_off.clone(),
                                     in_len=db.in_len.clone(), sa_idx=db.sa_idx.clone(),
                                     out_buf=torch.empty_like(db.out_buf), out_off=db.out_off.clone(),
                                     out_len=torch.empty_like(db.out_len)) for _ in range(R - 1)]
    t = nba_ipsec.SATable(p, max_batch=b.n)
    K = 200
    ring = t.ring([(*d.args(), b.n) for d in dbs]) if os.environ.get("AB_RING") else None
    def go(k_steps):
        if ring is not None:
            ring.run(k_steps // R)
            for k in range(k_steps %% R):
                t.process(*dbs[k].args(), n=b.n)
        else:
            for k in range(k_steps):
                t.process(*dbs[k %% R].args(), n=b.n)
    go(2 * R)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    go(K)
    e1.record()
    torch.cuda.synchronize()
    print(f"  cfg {cfg}: {e0.elapsed_time(e1) / K * 1e3:.2f} us/step (R={R})", flush=True)
    if ring is not None:
        ring.close()
    t.close()
    del dbs
'''


def main():
    libs = sys.argv[1:] or [os.path.join(ROOT, "paper_conf_eurosys_kimjlmsm15_b200", "libnba_ipsec.so")]
    for rep in range(2):
        for lib in libs:
            env = dict(os.environ, NBA_IPSEC_LIB=os.path.abspath(lib))
            print(f"{os.path.basename(lib)} (pass {rep}):", flush=True)
            subprocess.run([sys.executable, "-c", TIMER % ROOT], env=env, check=False)


if __name__ == "__main__":
    main()
