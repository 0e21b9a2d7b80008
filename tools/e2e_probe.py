"""Probe the host-buffer path: host time per call and step time for depth-2 pipelining."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import gen, nba_ipsec  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 2
c = gen.CONFIGS[cfg]
p = gen.make_sas(c["n_sa"], cfg_id=cfg)
b = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=cfg, layout="packed")
t = nba_ipsec.SATable(p, max_batch=c["n"])
in_bytes = int(b.in_off[-1]) + int(b.in_len[-1])
out_bytes = int(b.out_pool_bytes)
t.reserve_host_io(in_bytes, out_bytes)
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()  # noqa: E731
h_in = pin(b.in_buf)
h_off, h_len, h_sa = pin(b.in_off.view(np.int32)), pin(b.in_len.view(np.int16)), pin(b.sa_idx.view(np.int32))
h_ooff = pin(b.out_off.view(np.int32))
h_out = torch.zeros(out_bytes, dtype=torch.uint8).pin_memory()
h_olen = torch.zeros(b.n, dtype=torch.int16).pin_memory()
st = torch.cuda.Stream() if "--stream" in sys.argv else torch.cuda.current_stream()
print("stream", st, "in", in_bytes, "out", out_bytes)


def step():
    t.process_host(h_in, h_off, h_len, h_sa, h_out, h_ooff, h_olen, in_bytes, out_bytes, n=b.n, stream=st)


for _ in range(10):
    step()
t.host_wait(st)
torch.cuda.synchronize()
N = 100
t0 = time.perf_counter()
for _ in range(N):
    step()
t1 = time.perf_counter()
t.host_wait(st)
torch.cuda.synchronize()
t2 = time.perf_counter()
print(f"host time per call {(t1 - t0) / N * 1e6:.1f} us; wall per step {(t2 - t0) / N * 1e6:.1f} us")
# serial reference: sync after each step
t0 = time.perf_counter()
for _ in range(20):
    step()
    t.host_wait(st)
    torch.cuda.synchronize()
print(f"serialised per step {(time.perf_counter() - t0) / 20 * 1e6:.1f} us")
