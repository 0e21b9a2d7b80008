import sys, numpy as np
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen, device, nba_ipsec
for n in (3000, 65536):
    p = gen.make_sas(1024, cfg_id=4); b = gen.make_batch(n, "imix", 1024, cfg_id=4)
    o_out, o_len, _ = oracle.process_batch(oracle.make_sas(p), 1024, b, n_threads=8)
    t = nba_ipsec.SATable(p, device=0, max_batch=n)
    db = device.to_device(b, "cuda"); t.process(*db.args(), n=n)
    g_out, g_len = device.fetch(db)
    bad_len = np.nonzero(g_len != o_len)[0]
    print("n", n, "bad len", bad_len.size, bad_len[:5], g_len[bad_len[:5]], o_len[bad_len[:5]])
    nb = 0
    for i in range(n):
        a, L = int(b.out_off[i]), int(o_len[i])
        g, o = g_out[a:a+L], o_out[a:a+L]
        if not np.array_equal(g, o):
            d = np.nonzero(g != o)[0]
            if nb < 8: print("pkt", i, "D", b.in_len[i], "L", L, "ndiff", d.size, "first", d[:6], "last", d[-3:])
            nb += 1
    print("bad pkts", nb)
