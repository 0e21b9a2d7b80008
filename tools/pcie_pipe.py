"""Copy-only pipeline with the e2e byte pattern (5 H2D + 2 D2H per step, two
staging slots, separate copy streams): the PCIe ceiling of the host path."""
import time
import torch
N_IN, N_OUT, N = 3276800, 7471120, 65536
h_in = torch.ones(N_IN, dtype=torch.uint8).pin_memory()
h_meta = [torch.ones(N * 4, dtype=torch.uint8).pin_memory() for _ in range(3)] + \
         [torch.ones(N * 2, dtype=torch.uint8).pin_memory()]
h_out = torch.zeros(N_OUT, dtype=torch.uint8).pin_memory()
h_ol = torch.zeros(N * 2, dtype=torch.uint8).pin_memory()
slots = [dict(i=torch.empty(N_IN, dtype=torch.uint8, device="cuda"),
              m=[torch.empty(x.numel(), dtype=torch.uint8, device="cuda") for x in h_meta],
              o=torch.empty(N_OUT, dtype=torch.uint8, device="cuda"),
              ol=torch.empty(N * 2, dtype=torch.uint8, device="cuda"),
              ev_in=torch.cuda.Event(), ev_out=torch.cuda.Event()) for _ in range(2)]
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def step(k, with_meta=True):
    sl = slots[k % 2]
    s1.wait_event(sl["ev_out"])
    with torch.cuda.stream(s1):
        sl["i"].copy_(h_in, non_blocking=True)
        if with_meta:
            for d, h in zip(sl["m"], h_meta):
                d.copy_(h, non_blocking=True)
        sl["ev_in"].record(s1)
    s2.wait_event(sl["ev_in"])
    with torch.cuda.stream(s2):
        h_out.copy_(sl["o"], non_blocking=True)
        if with_meta:
            h_ol.copy_(sl["ol"], non_blocking=True)
        sl["ev_out"].record(s2)


for wm in (True, False):
    for k in range(10):
        step(k, wm)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for k in range(100):
        step(k, wm)
    torch.cuda.synchronize()
    print(f"copy pipeline (meta={wm}): {(time.perf_counter() - t0) / 100 * 1e6:.1f} us/step")
