import os, sys
sys.path.insert(0, "/root/repo")
import torch
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec
sys.path.insert(0, "/root/repo/tools")
from ab_merge import timed
for n, size in ((64, 64), (1024, 64), (8192, 64), (8192, "imix"), (32768, 64)):
    p = gen.make_sas(1024, cfg_id=2)
    b = gen.make_batch(n, size, 1024, cfg_id=2)
    db = device.to_device(b, "cuda")
    tm = nba_ipsec.SATable(p, max_batch=n)
    os.environ["NBA_IPSEC_NO_MERGE"] = "1"
    t2 = nba_ipsec.SATable(p, max_batch=n)
    del os.environ["NBA_IPSEC_NO_MERGE"]
    print(f"n={n} size={size}: merged {timed(tm, db, n):.1f} us, two-kernel {timed(t2, db, n):.1f} us")
