#!/usr/bin/env python
"""Same-box A/B of compile-time variants of the batch ring, and a phase trace.

    python tools/ring_ab.py build NAME=DEF1,DEF2 ...      (CPU: nvcc only -> build/variants/NAME.so)
    python tools/ring_ab.py run [sizes...]                (GPU: bench protocol per variant, 2 passes)
    python tools/ring_ab.py trace [sizes...]              (GPU: needs build/variants/trace.so,
                                                           built with NBA_RING_TRACE=1)

`run` times every variant (and the default library as `base`) in a fresh
process through the NBA_IPSEC_LIB override with the bench's protocol: R device
copies of a full-size 65,536-packet batch (1024 SAs), >= 2R warm-up batches,
then K = 200 batches in ONE nba_ipsec_ring_run_batches call between one CUDA
event pair.  Passes are interleaved to expose drift.

`trace` prints, per size, the median over batches and CTAs of each phase of
the software-pipelined ring (k_fused_ring_pipe): barrier seen, scans + polls
done, lanes done, prologue warps' arrival for the next batch, iteration end,
relative to the iteration start -- what sits on the per-batch critical path."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
VDIR = os.path.join(ROOT, "build", "variants")
sys.path.insert(0, ROOT)

TIMER = r'''
import os, sys, json
sys.path.insert(0, %(root)r)
import numpy as np, torch
from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec, shard
K = %(k)d
out = {}
for size in %(sizes)r:
    cfg = {64: 2, 1514: 3, "imix": 4}.get(size, 5)
    p, b = shard.rank_workload(cfg, 65536, size, 1024, 0, 1)
    t = nba_ipsec.SATable(p, max_batch=65536)
    d0 = device.to_device(b, "cuda")
    R = device.ring_slot_count(b.in_len, b.n, torch.cuda.get_device_properties(0).L2_cache_size)
    dbs = [d0] + [device.clone(d0) for _ in range(R - 1)]
    ring = t.ring([(*d.args(), b.n) for d in dbs])
    ring.run_batches(max(40, 4 * R)); torch.cuda.synchronize()
    if %(trace)r:
        G = 148
        ts = torch.zeros(K * G * 16 + 4 * 4 * 448 * 8, dtype=torch.int64, device="cuda")
        ring.set_timestamps(ts)
        ring.run_batches(K); torch.cuda.synchronize()
        tsn = ts.cpu().numpy().astype(np.int64)
        vall = tsn[:K * G * 16].reshape(K, G, 16)
        # lane timelines of batches 0..3 (CTAs 0..3): clock64 segments (setup, AES step 0,
        # emission, SHA block 0, rest) and globaltimer start / end of esp_packet
        ld = tsn[K * G * 16:].reshape(4, 4, 448, 8)
        lanes_tl = {}
        for bb in range(4):
            x = ld[bb].reshape(-1, 8)
            x = x[x[:, 7] > 0]
            if not len(x):
                continue
            it0 = vall[bb, :4, 0].min()
            lanes_tl[bb] = {"n": int(len(x)), "seg_cycles_median": [int(np.median(x[:, j])) for j in range(5)],
                            "seg_cycles_p90": [int(np.percentile(x[:, j], 90)) for j in range(5)],
                            "start_us_p10_50_90": [round(float(np.percentile((x[:, 6] - it0) / 1e3, q)), 2) for q in (10, 50, 90)],
                            "dur_us_p10_50_90": [round(float(np.percentile((x[:, 7] - x[:, 6]) / 1e3, q)), 2) for q in (10, 50, 90)]}
        k0 = vall[0, :, 15].min()                 # the run's first CTA start
        su = lambda a: round(float(np.median((a - k0) / 1e3)), 2)  # noqa: E731
        startup = {"cta_start": su(vall[0, :, 15]), "b0_meta_issued": su(vall[0, :, 13]),
                   "b0_prologue_done": su(vall[0, :, 14]), "tables_landed": su(vall[1, :, 15]),
                   "it0_start": su(vall[0, :, 0]), "it0_barrier_seen": su(vall[0, :, 1]),
                   "it0_polls_done": su(vall[0, :, 2]), "it0_lanes_done": su(vall[0, :, 3]),
                   "it0_end": su(vall[0, :, 5]), "it1_end": su(vall[1, :, 5]), "lanes": lanes_tl}
        v = vall[2:-1]                            # skip start-up, last
        rel = (v - v[:, :, :1]) / 1e3
        names = ["start", "barrier_seen", "polls_done", "lanes_done", "prologue_arrived",
                 "iter_end", "early_keys_done", "pseq_polls_done", "pro_meta", "pro_ranked",
                 "pro_counts", "pro_perm", "pro_lpt"]
        ok = lambda i: bool(np.all(v[:, :, i] > 0))
        med = {n: round(float(np.median(rel[:, :, i])), 2) for i, n in enumerate(names) if i and ok(i)}
        p90 = {n: round(float(np.percentile(rel[:, :, i], 90)), 2) for i, n in enumerate(names) if i and ok(i)}
        lanes = rel[:, :, 3]
        order = np.argsort(-np.median(lanes, axis=0))[:6]
        p90["slowest_ctas_lanes_us"] = [(int(c), round(float(np.median(lanes[:, c])), 2)) for c in order]
        p90["lanes_done_max_over_ctas"] = round(float(np.median(np.max(lanes, axis=1))), 2)
        it = np.diff(v[:, 0, 0]) / 1e3
        out[str(size)] = {"median_us": med, "p90_us": p90, "iter_us": float(np.median(it)), "startup": startup}
    else:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); ring.run_batches(K); e1.record(); torch.cuda.synchronize()
        out[str(size)] = round(e0.elapsed_time(e1) * 1e3 / K, 2)
    ring.close(); t.close(); del dbs
print(json.dumps(out), flush=True)
'''


def run_one(lib, sizes, k, trace):
    env = dict(os.environ)
    if lib:
        env["NBA_IPSEC_LIB"] = lib
    code = TIMER % {"root": ROOT, "sizes": sizes, "k": k, "trace": trace}
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True)
    if r.returncode:
        return "FAILED: " + r.stderr[-600:]
    return r.stdout.strip()


def main():
    cmd = sys.argv[1]
    args = sys.argv[2:]
    if cmd == "build":
        from paper_conf_eurosys_kimjlmsm15_b200 import build
        os.makedirs(VDIR, exist_ok=True)
        for spec in args:
            name, _, defs = spec.partition("=")
            d = [x for x in defs.split(",") if x]
            print(name, build.build(out=os.path.join(VDIR, name + ".so"), defines=d), flush=True)
        return
    sizes = [x if x == "imix" else int(x) for x in args] or [64, 1514, "imix"]
    if cmd == "trace":
        for f in sorted(os.listdir(VDIR)):
            if f.endswith("trace.so"):
                print(f[:-3], run_one(os.path.join(VDIR, f), sizes, 50, True), flush=True)
        return
    names = sorted(f[:-3] for f in os.listdir(VDIR) if f.endswith(".so") and not f.endswith("trace.so")) \
        if os.path.isdir(VDIR) else []
    for rep in range(int(os.environ.get("AB_PASSES", "2"))):
        print(f"pass {rep} base", run_one(None, sizes, 200, False), flush=True)
        for n in names:
            print(f"pass {rep} {n}", run_one(os.path.join(VDIR, n + ".so"), sizes, 200, False),
                  flush=True)


if __name__ == "__main__":
    main()
