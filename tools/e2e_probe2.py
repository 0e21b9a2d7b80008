"""Where does the host-buffer path lose its copy overlap?  The
process_batch_host stream structure rebuilt in Python (H2D stream, compute
stream, D2H stream, DEPTH staging slots) with the compute step being (a)
nothing, (b) the library's device path (cooperative one-kernel launch), (c) a
torch kernel of similar duration; 64 B config, us/step."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

DEPTH = int(sys.argv[1]) if len(sys.argv) > 1 else 2
p = gen.make_sas(1024, cfg_id=2)
b = gen.make_batch(65536, 64, 1024, cfg_id=2, layout="packed")
t = nba_ipsec.SATable(p, max_batch=b.n)
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()  # noqa: E731
h_in = [pin(b.in_buf), pin(b.in_off.view(np.int32)), pin(b.in_len.view(np.int16)),
        pin(b.sa_idx.view(np.int32)), pin(b.out_off.view(np.int32))]
h_out = torch.empty(b.out_pool_bytes, dtype=torch.uint8).pin_memory()
h_ol = torch.empty(b.n, dtype=torch.int16).pin_memory()
slots = []
for _ in range(DEPTH):
    d = device.to_device(b, "cuda")
    slots.append(dict(d=d, ev_in=torch.cuda.Event(), ev_done=torch.cuda.Event(),
                      ev_out=torch.cuda.Event()))
s_h, s_c, s_d = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
x = torch.randn(1 << 22, device="cuda")


def step(k, mode):
    sl = slots[k % DEPTH]
    d = sl["d"]
    s_h.wait_event(sl["ev_out"])
    with torch.cuda.stream(s_h):
        for dst, src in zip((d.in_buf, d.in_off, d.in_len, d.sa_idx, d.out_off), h_in):
            dst[:src.numel()].copy_(src, non_blocking=True)
        sl["ev_in"].record(s_h)
    s_c.wait_event(sl["ev_in"])
    with torch.cuda.stream(s_c):
        if mode == "lib":
            t.process(*d.args(), n=b.n, stream=s_c)
        elif mode == "torch":
            for _ in range(3):
                x.mul_(1.0001)
        sl["ev_done"].record(s_c)
    s_d.wait_event(sl["ev_done"])
    with torch.cuda.stream(s_d):
        h_out.copy_(d.out_buf[:h_out.numel()], non_blocking=True)
        h_ol.copy_(d.out_len[:b.n], non_blocking=True)
        sl["ev_out"].record(s_d)


for mode in ("none", "torch", "lib", "none", "lib"):
    for k in range(10):
        step(k, mode)
    torch.cuda.synchronize()
    K = 100
    t0 = time.perf_counter()
    for k in range(K):
        step(k, mode)
    torch.cuda.synchronize()
    print(f"depth {DEPTH} compute={mode}: {(time.perf_counter() - t0) / K * 1e6:.1f} us/step", flush=True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(s_c)
for _ in range(3):
    x.mul_(1.0001)
e1.record(s_c)
torch.cuda.synchronize()
print(f"torch compute alone: {e0.elapsed_time(e1) * 1e3:.1f} us")
