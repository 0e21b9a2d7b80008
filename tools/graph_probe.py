"""CUDA-graph replay of the one-kernel path (device-side barrier base / epoch):
R batch slots captured once as R cooperative kernel nodes, replayed; vs the same
launches from the stream.  Checks that both give identical output and SA
counters, then times each (64 B config, back to back, L2-cold rotation)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
size = {2: 64, 3: 1514, 4: "imix"}[cfg]
p = gen.make_sas(1024, cfg_id=cfg)
b = gen.make_batch(65536, size, 1024, cfg_id=cfg)
db = device.to_device(b, "cuda")
L2 = torch.cuda.get_device_properties(0).L2_cache_size
R = max(2, -(-2 * L2 // (int(b.in_len.astype(np.int64).sum()) + b.n * 451)))
dbs = [db] + [device.DeviceBatch(n=db.n, in_buf=db.in_buf.clone(), in_off=db.in_off.clone(),
                                 in_len=db.in_len.clone(), sa_idx=db.sa_idx.clone(),
                                 out_buf=torch.zeros_like(db.out_buf), out_off=db.out_off.clone(),
                                 out_len=torch.zeros_like(db.out_len)) for _ in range(R - 1)]
ta = nba_ipsec.SATable(p, max_batch=b.n)
tb = nba_ipsec.SATable(p, max_batch=b.n)
s = torch.cuda.Stream()
# warm both tables identically (one batch each) outside the graph
with torch.cuda.stream(s):
    ta.process(*dbs[0].args(), n=b.n, stream=s)
    tb.process(*dbs[0].args(), n=b.n, stream=s)
s.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=s):
    for d in dbs:
        ta.process(*d.args(), n=b.n, stream=s)
torch.cuda.synchronize()
# correctness: 2 replays on ta vs 2 rounds of stream launches on tb
for _ in range(2):
    g.replay()
torch.cuda.synchronize()
out_a = [d.out_buf.clone() for d in dbs]
len_a = [d.out_len.clone() for d in dbs]
for _ in range(2):
    for d in dbs:
        tb.process(*d.args(), n=b.n)
torch.cuda.synchronize()
same = all(torch.equal(x, d.out_buf) for x, d in zip(out_a, dbs)) and \
    all(torch.equal(x, d.out_len) for x, d in zip(len_a, dbs))
print("graph == stream launches:", same, " SA seq equal:", bool(np.array_equal(ta.sa_seq(), tb.sa_seq())),
      " R =", R, flush=True)
K = 20
for name in ("stream", "graph", "stream", "graph"):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    with torch.cuda.stream(s):
        for _ in range(K):
            if name == "graph":
                g.replay()
            else:
                for d in dbs:
                    ta.process(*d.args(), n=b.n, stream=s)
    e1.record(s)
    torch.cuda.synchronize()
    print(f"{name}: {e0.elapsed_time(e1) / (K * R) * 1e3:.2f} us/batch", flush=True)
