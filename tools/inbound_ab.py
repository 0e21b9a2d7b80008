#!/usr/bin/env python
"""ESP inbound ring forms side by side (GPU), each forced: the CUDA-graph ring of
one-kernel launches, the plain persistent ring and the software-pipelined one, on the
bench's inbound protocol (R ESP batches from R consecutive outbound batches,
each rotation through nba_ipsec_ring_run_batches, windows reset per rotation),
K = 100 batches between one CUDA event pair, per size; optionally per library
variant (NBA_IPSEC_LIB).

    python tools/inbound_ab.py [sizes...]"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CODE = r'''
import os, sys, json
sys.path.insert(0, %(root)r)
import numpy as np, torch
from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec, shard
K = 100
out = {}
for size in %(sizes)r:
    cfg = {64: 2, 1514: 3, "imix": 4}.get(size, 5)
    p, b = shard.rank_workload(cfg, 65536, size, 1024, 0, 1)
    db = device.to_device(b, "cuda")
    R = device.ring_slot_count(b.in_len, b.n, torch.cuda.get_device_properties(0).L2_cache_size)
    t_out = nba_ipsec.SATable(p, max_batch=65536)
    esp = []
    for _ in range(R):
        ob, ol = torch.empty_like(db.out_buf), torch.zeros_like(db.out_len)
        t_out.process(db.in_buf, db.in_off, db.in_len, db.sa_idx, ob, db.out_off, ol, n=b.n)
        esp.append((ob, ol, torch.empty_like(db.out_buf), torch.zeros_like(db.out_len)))
    torch.cuda.synchronize(); t_out.close()
    t = nba_ipsec.SATable(p, max_batch=65536)
    t.enable_inbound()
    ring = t.ring_inbound([(e[0], db.out_off, e[1], db.sa_idx, e[2], db.out_off, e[3], None, b.n) for e in esp])
    def run(k):
        left = k
        while left:
            if ring.cursor == 0:
                t.reset_inbound()
            nb = min(left, R - ring.cursor)
            ring.run_batches(nb)
            left -= nb
    run(2 * R); torch.cuda.synchronize()
    if %(trace)r:
        G = 148
        ts = torch.zeros(R * G * 16, dtype=torch.int64, device="cuda")
        ring.set_timestamps(ts)
        t.reset_inbound(); ring.run_batches(R); torch.cuda.synchronize()
        v = ts.cpu().numpy().reshape(R, G, 16).astype(np.int64)[1:-1]
        t0 = v[:, :, :1].min(axis=1, keepdims=True)       # the batch's first CTA start
        v = np.where(v > 0, v, t0)                          # (stamps a form does not take)
        rel = (v - t0) / 1e3
        # pipelined ring: 1 / 8 are the side warps' row scans of the PREVIOUS
        # batch during this one (SB1 passed, scans done), 9 the lane warps'
        # decisions of the previous batch
        names = {0: "iter_start", 1: "prev_sb1_passed", 3: "lanes_done", 4: "side_done", 5: "iter_end",
                 6: "tile_done", 8: "prev_row_scans_done", 9: "prev_decisions_done",
                 10: "pro_formats_done", 11: "pro_stored", 12: "pro_sorted"}
        out[str(size)] = {n: [round(float(np.median(rel[:, :, i])), 2),
                              round(float(np.median(np.max(rel[:, :, i], axis=1))), 2)]
                          for i, n in names.items()}
        lanes = rel[:, :, 3]
        order = np.argsort(-np.median(lanes, axis=0))[:6]
        out[str(size)]["slowest_ctas_lanes_us"] = [(int(c), round(float(np.median(lanes[:, c])), 2))
                                                  for c in order]
        ring.close(); t.close(); del esp
        continue
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); run(K); e1.record(); torch.cuda.synchronize()
    c = t.in_counters()
    out[str(size)] = {"us": round(e0.elapsed_time(e1) * 1e3 / K, 2), "form": ring.form,
                      "all_ok": c["pkts_ok"] == c["batches"] * b.n}
    ring.close(); t.close(); del esp
print(json.dumps(out), flush=True)
'''


def main():
    if sys.argv[1:2] == ["trace"]:
        sizes = [x if x == "imix" else int(x) for x in sys.argv[2:]] or [64, 1514, "imix"]
        env = dict(os.environ, NBA_IPSEC_LIB=os.path.join(ROOT, "build", "variants", "trace.so"),
                   NBA_IPSEC_RING_IN_PIPE="1")
        r = subprocess.run([sys.executable, "-c", CODE % {"root": ROOT, "sizes": sizes, "trace": True}],
                           env=env, capture_output=True, text=True)
        print("trace", r.stdout.strip() if r.returncode == 0 else "FAILED " + r.stderr[-800:])
        return
    sizes = [x if x == "imix" else int(x) for x in sys.argv[1:]] or [64, 1514, "imix"]
    for rep in range(2):
        for form in ("graph", "persistent", "pipelined"):
            env = dict(os.environ)
            if form == "graph":
                env["NBA_IPSEC_RING_IN_PIPE"] = "0"
            if form == "persistent":
                env["NBA_IPSEC_RING_IN_PERSIST"] = "1"
            if form == "pipelined":
                env["NBA_IPSEC_RING_IN_PIPE"] = "1"
            r = subprocess.run([sys.executable, "-c", CODE % {"root": ROOT, "sizes": sizes, "trace": False}], env=env,
                               capture_output=True, text=True)
            print(f"pass {rep} {form}", r.stdout.strip() if r.returncode == 0 else "FAILED " + r.stderr[-500:],
                  flush=True)


if __name__ == "__main__":
    main()
