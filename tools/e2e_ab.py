"""e2e (host-buffer path) A/B of library variants: the bench's run_e2e
protocol (pinned host buffers, nba_ipsec_process_batch_host every step,
copy-in / kernels / copy-out pipelined), configs 2-4, one fresh process per
variant via NBA_IPSEC_LIB.   python tools/e2e_ab.py lib.so ..."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CODE = r'''
import os, sys
sys.path.insert(0, %r)
import numpy as np, torch
from paper_conf_eurosys_kimjlmsm15_b200 import gen, nba_ipsec
if os.environ.get("E2E_NUMA"):
    import pynvml
    pynvml.nvmlInit()
    pynvml.nvmlDeviceSetCpuAffinity(pynvml.nvmlDeviceGetHandleByIndex(0))
    print("  affinity", sorted(os.sched_getaffinity(0))[:4], "...", len(os.sched_getaffinity(0)), "cpus")
for cfg, size in ((2, 64),):
    p = gen.make_sas(1024, cfg_id=cfg)
    b = gen.make_batch(65536, size, 1024, cfg_id=cfg, layout="packed")
    t = nba_ipsec.SATable(p, max_batch=b.n)
    if os.environ.get("E2E_PIPE"): t.set_pipeline(int(os.environ["E2E_PIPE"]))
    ib = int(b.in_off[-1]) + int(b.in_len[-1]); ob = int(b.out_pool_bytes)
    t.reserve_host_io(ib, ob)
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
    h = (pin(b.in_buf), pin(b.in_off.view(np.int32)), pin(b.in_len.view(np.int16)),
         pin(b.sa_idx.view(np.int32)), torch.empty(ob, dtype=torch.uint8).pin_memory(),
         pin(b.out_off.view(np.int32)), torch.empty(b.n, dtype=torch.int16).pin_memory())
    st = torch.cuda.Stream() if os.environ.get("E2E_OWN_STREAM") else torch.cuda.current_stream()
    step = lambda: t.process_host(*h, ib, ob, n=b.n, stream=st)
    for _ in range(5): step()
    t.host_wait(st); torch.cuda.synchronize()
    K = 100
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    import time
    e0.record(st)
    h0 = time.perf_counter()
    for _ in range(K): step()
    h1 = time.perf_counter()
    t.host_wait(st); e1.record(st); torch.cuda.synchronize()
    print(f"  host enqueue {1e6 * (h1 - h0) / K:.1f} us/step", flush=True)
    ms = e0.elapsed_time(e1) / K
    gbps = 8.0 * float(b.frame_len.astype(np.float64).sum()) / (ms * 1e-3) / 1e9
    print(f"  cfg {cfg}: {ms * 1e3:.1f} us/step  {gbps:.1f} Gbps  (h2d {ib + 14 * b.n} B, d2h {ob + 2 * b.n} B)", flush=True)
    t.close()
'''
for lib in sys.argv[1:]:
    print(os.path.basename(lib), flush=True)
    subprocess.run([sys.executable, "-c", CODE % ROOT], env=dict(os.environ, NBA_IPSEC_LIB=os.path.abspath(lib)))
