#!/usr/bin/env python
"""PCIe copy rates on the box (GPU): H2D alone, D2H alone, both at once on two
streams, at the e2e step's sizes (64 B config), pinned host memory; then the
e2e loop itself (nba_ipsec_process_batch_host) for comparison.

    python tools/pcie_probe.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

K = 50
H2D, D2H = 4194304 + 65536 * 14, 6881296
hi = torch.empty(H2D, dtype=torch.uint8).pin_memory()
ho = torch.empty(D2H, dtype=torch.uint8).pin_memory()
di = torch.empty(H2D, dtype=torch.uint8, device="cuda")
do = torch.empty(D2H, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
out = {}


def timed(fn):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e-3


def h2d():
    with torch.cuda.stream(s1):
        for _ in range(K):
            di.copy_(hi, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)


def d2h():
    with torch.cuda.stream(s2):
        for _ in range(K):
            ho.copy_(do, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s2)


def both():
    torch.cuda.current_stream()
    with torch.cuda.stream(s1):
        for _ in range(K):
            di.copy_(hi, non_blocking=True)
    with torch.cuda.stream(s2):
        for _ in range(K):
            ho.copy_(do, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)
    torch.cuda.current_stream().wait_stream(s2)


t = timed(h2d)
out["h2d_GBps"] = round(H2D * K / t / 1e9, 1)
t = timed(d2h)
out["d2h_GBps"] = round(D2H * K / t / 1e9, 1)
t = timed(both)
out["both_us_per_step"] = round(t / K * 1e6, 1)
out["both_h2d_GBps"] = round(H2D * K / t / 1e9, 1)
out["both_d2h_GBps"] = round(D2H * K / t / 1e9, 1)
out["serial_us_per_step"] = round((H2D / (out["h2d_GBps"] * 1e9) + D2H / (out["d2h_GBps"] * 1e9)) * 1e6, 1)
props = torch.cuda.get_device_properties(0)
out["async_engines"] = getattr(props, "async_engine_count", None)
print(json.dumps(out), flush=True)

# the e2e loop (bench.run_e2e's protocol) with the library (NBA_IPSEC_LIB picks a variant)
import numpy as np  # noqa: E402
from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec, shard  # noqa: E402
p, b = shard.rank_workload(2, 65536, 64, 1024, 0, 1, layout="packed", out_pad=53)
tb = nba_ipsec.SATable(p, device=0, max_batch=65536)
in_bytes = int(b.in_off[-1]) + int(b.in_len[-1])
out_bytes = int(b.out_pool_bytes)
tb.reserve_host_io(in_bytes, out_bytes)
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()  # noqa: E731
h_in = pin(b.in_buf)
h_off, h_len, h_sa = pin(b.in_off.view(np.int32)), pin(b.in_len.view(np.int16)), pin(b.sa_idx.view(np.int32))
h_ooff = pin(b.out_off.view(np.int32))
h_out = torch.empty(out_bytes, dtype=torch.uint8).pin_memory()
h_olen = torch.empty(b.n, dtype=torch.int16).pin_memory()
st = torch.cuda.current_stream()


def e2e():
    for _ in range(K):
        tb.process_host(h_in, h_off, h_len, h_sa, h_out, h_ooff, h_olen, in_bytes, out_bytes, n=b.n, stream=st)
    tb.host_wait(st)


import time  # noqa: E402
e2e()
torch.cuda.synchronize()
c0 = time.perf_counter()
e2e()
cpu = time.perf_counter() - c0
torch.cuda.synchronize()
t = timed(e2e)
print(json.dumps({"lib": os.environ.get("NBA_IPSEC_LIB", "default"), "e2e_us_per_step": round(t / K * 1e6, 1),
                  "submit_cpu_us_per_step": round(cpu / K * 1e6, 1),
                  "in_bytes": in_bytes, "out_bytes": out_bytes}), flush=True)

# the same pipeline with plain torch copies (no kernel): three streams, two
# staging slots, the e2e step's copy list -- what the copy engines give
s3 = torch.cuda.Stream()
meta = [torch.empty(65536 * w, dtype=torch.uint8).pin_memory() for w in (4, 4, 4, 2)]
slots = []
for _ in range(2):
    slots.append({"in": torch.empty(in_bytes, dtype=torch.uint8, device="cuda"),
                  "meta": [torch.empty(m.numel(), dtype=torch.uint8, device="cuda") for m in meta],
                  "out": torch.empty(out_bytes, dtype=torch.uint8, device="cuda"),
                  "olen": torch.empty(65536 * 2, dtype=torch.uint8, device="cuda"),
                  "ev_in": torch.cuda.Event(), "ev_done": torch.cuda.Event(), "ev_out": torch.cuda.Event()})
h_in2 = torch.empty(in_bytes, dtype=torch.uint8).pin_memory()
h_out2 = torch.empty(out_bytes, dtype=torch.uint8).pin_memory()
h_olen2 = torch.empty(65536 * 2, dtype=torch.uint8).pin_memory()


dmeta = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in
         (b.in_off.view(np.int32), b.in_len.view(np.int16), b.sa_idx.view(np.int32), b.out_off.view(np.int32))]
dolen = torch.empty(b.n, dtype=torch.int16, device="cuda")
for sl in slots:
    sl["in"].copy_(torch.from_numpy(b.in_buf[:in_bytes]))


def emul(big_only=False, kernel=False):
    for k in range(K):
        sl = slots[k % 2]
        with torch.cuda.stream(s1):
            s1.wait_event(sl["ev_out"])
            sl["in"].copy_(h_in2, non_blocking=True)
            if not big_only:
                for d, h in zip(sl["meta"], meta):
                    d.copy_(h, non_blocking=True)
            sl["ev_in"].record(s1)
        with torch.cuda.stream(s2):
            s2.wait_event(sl["ev_in"])
            if kernel:
                tb.process(sl["in"], dmeta[0], dmeta[1], dmeta[2], sl["out"], dmeta[3], dolen, n=b.n, stream=s2)
            sl["ev_done"].record(s2)
        with torch.cuda.stream(s3):
            s3.wait_event(sl["ev_done"])
            h_out2.copy_(sl["out"], non_blocking=True)
            if not big_only:
                h_olen2.copy_(sl["olen"], non_blocking=True)
            sl["ev_out"].record(s3)
    torch.cuda.current_stream().wait_stream(s3)


t = timed(emul)
t2 = timed(lambda: emul(True))
t3 = timed(lambda: emul(False, True))
t4 = timed(lambda: emul(True, True))
print(json.dumps({"torch_pipeline_us_per_step": round(t / K * 1e6, 1),
                  "torch_pipeline_big_copies_only_us": round(t2 / K * 1e6, 1),
                  "with_kernel_us": round(t3 / K * 1e6, 1),
                  "big_copies_with_kernel_us": round(t4 / K * 1e6, 1)}), flush=True)
