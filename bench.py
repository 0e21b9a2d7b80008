#!/usr/bin/env python
"""Benchmark: IPsec ESP outbound throughput (Gbps, Mpps) per packet size on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 2|3|4] [--impl ours|reference]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N

One step = one batch of 65,536 packets per GPU through the whole hot path
(prologue, gather + ESP encapsulation, AES-128-CTR, HMAC-SHA1-96,
scatter) with inputs resident in HBM.  The headline (`value`) is BASELINE.json
configs[1] (64-B frames, 1024 SAs); configs[2] (1514 B), configs[3] (IMIX) and
the configs[4] sweep (64 / 128 / 256 / 512 / 1024 / 1514 B + IMIX) are measured
in the same run (`gbps_by_size`).  Multi-GPU (configs[4] at 2/4/8 GPUs): SA-hash
sharding (GPU g owns SAs s = g mod N), weak scaling, no data-path
collective; NCCL only reduces counters and takes the max elapsed time.
`--gpus N` without a torchrun environment re-launches itself under torchrun
(one process per GPU).

Timing: the K timed batches run back to back on the launching
stream between one CUDA event pair (barrier + synchronize on both sides, max
over ranks), rotating over R device copies of the batch whose touched bytes
exceed 2x the L2 (every batch starts L2-cold); EVERY timed batch goes through
the library's batch ring (nba_ipsec_ring_run_batches: one persistent launch for
all K).  A second pass records per-batch device timestamps (median / p10 / p90).
Beside it: the same K batches as plain process_batch launches, as CUDA-graph
replay, and one batch at a time with L2 flushed.

Gbps = 8 * sum(frame bytes L) / t (reading A18, frames excluding FCS); Mpps =
packets / t; ESP-payload Gbps = 8 * sum(D) / t.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import gen, shard  # noqa: E402

METRIC = "IPsec ESP throughput Gbps & Mpps per packet size at 1/2/4/8 B200; % roofline"
N_SA_TOTAL = 1024
PKTS_PER_GPU = 65536
CFG_SIZE = {2: 64, 3: 1514, 4: "imix"}
SWEEP = [(2, 64), (5, 128), (5, 256), (5, 512), (5, 1024), (3, 1514), (4, "imix")]   # configs[4]
SM_COUNT = 148


# --------------------------------------------------------------------------- utils
def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return {"hbm_gbs": float(d["hbm_gbs"]), "sm_max_mhz": float(d.get("sm_max_mhz", 1965.0)),
                "source": "measured (MEASURED_PEAKS.json)"}
    except Exception:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0, "source": "fallback (B200_PROFILING.md)"}


def gpu_lead(torch, us: float = 100.0):
    """A sleep kernel just before a timed region's start event: the GPU is busy
    while the host enqueues the start event and the launches, so the events
    measure device time, not the host's enqueue latency (the GIL, the NVML
    sampler thread) -- with K = 20 ring batches (~0.5 ms) that jitter was
    ~40 us per run (tools/ring_startup.py)."""
    torch.cuda._sleep(int(us * 2000))       # cycles at <= 2 GHz: >= `us` microseconds


class ClockSampler:
    """Samples SM clock + throttle reasons with NVML during the timed region."""

    def __init__(self, gpu_index: int, period_s: float = 0.001):
        self.idx, self.period = gpu_index, period_s
        self.samples, self.reasons = [], set()
        self._stop = threading.Event()
        self.max_mhz = None
        self._t = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.idx)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            names = {
                "hw_slowdown": getattr(pynvml, "nvmlClocksEventReasonHwSlowdown", 0x8),
                "hw_thermal_slowdown": getattr(pynvml, "nvmlClocksEventReasonHwThermalSlowdown", 0x40),
                "sw_thermal_slowdown": getattr(pynvml, "nvmlClocksEventReasonSwThermalSlowdown", 0x20),
                "sw_power_cap": getattr(pynvml, "nvmlClocksEventReasonSwPowerCap", 0x4),
                "hw_power_brake_slowdown": getattr(pynvml, "nvmlClocksEventReasonHwPowerBrakeSlowdown", 0x80),
            }

            def run():
                while not self._stop.is_set():
                    try:
                        self.samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                        r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                        for k, bit in names.items():
                            if r & bit:
                                self.reasons.add(k)
                    except Exception:
                        pass
                    time.sleep(self.period)

            self._t = threading.Thread(target=run, daemon=True)
            self._t.start()
        except Exception as e:  # NVML unavailable: record why
            self.reasons.add(f"nvml_unavailable:{type(e).__name__}")
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        return {"sm_mhz": float(statistics.median(self.samples)) if self.samples else None,
                "sm_max_mhz": float(self.max_mhz) if self.max_mhz else None,
                "samples": len(self.samples), "reasons": sorted(self.reasons)}


def frame_bits(b):
    return 8.0 * float(np.asarray(b.frame_len, np.float64).sum())


def work_model(b):
    """Algorithmic work of one batch: per
    valid packet AES blocks ceil(C/16), SHA-1 compressions (inner
    ceil((C+25)/64) + outer 1; the ipad/opad blocks are precomputed at SA
    setup), bytes read D and written 48 + C, 16 B of metadata."""
    D = b.in_len.astype(np.int64)
    ok = (D >= 20) & (D <= 1500) & (b.sa_idx < 2**31)
    D = D[ok]
    C = D + ((-(D + 2)) % 4) + 2
    return {
        "packets": int(ok.sum()),
        "aes_blocks": int(((C + 15) // 16).sum()),
        "sha1_compressions": int(((16 + C + 8) // 64 + 1 + 1).sum()),
        "bytes_in": int(D.sum()),
        "bytes_out": int((48 + C).sum()),
        "hbm_bytes": int(D.sum() + (48 + C).sum() + 16 * ok.sum()),
    }


# Per-unit work, SASS-derived (tools/sass_hist.py over the shipped
# k_fused_ring_roles -- the headline's kernel; k_fused_ring_pipe's counts,
# profiles/r02_sass_hist.txt, differ by < 1% -- committed as
# profiles/r02d_sass_hist.txt): instructions per AES-128 block (a quarter of the
# 4-block step, round loop x 7) and per SHA-1 compression, by issuing pipe.
# Fallbacks = the r02 counts.
SASS_HIST = os.path.join(ROOT, "profiles", "r02d_sass_hist.txt")
SASS_FALLBACK = {"aes_block": {"alu": 217.75, "fma": 19.5, "smem": 136.75},
                 "sha1_compression": {"alu": 434, "fma": 244, "smem": 0}}
ALU_LANES_PER_CLK_SM = 64          # B300_MICROARCH "Pipe rates"; microbenchmarked 63.9 on B200
LDS_LANES_PER_CLK_SM = 32          # 128 B/clk/SM shared crossbar (B300_MICROARCH LDS/STS)


def sass_units():
    try:
        for line in open(SASS_HIST):
            if line.startswith("JSON "):
                d = json.loads(line[5:])
                return {"aes_block": d["aes_block"], "sha1_compression": d["sha1_compression"],
                        "source": "profiles/r02d_sass_hist.txt"}
    except Exception:
        pass
    return dict(SASS_FALLBACK, source="fallback constants (r02 SASS counts)")


def roofline(ms_per_batch, w, peaks, units):
    """ALU, LDS and HBM fractions of the fused kernel side by side; `bound` is
    the resource the kernel is closest to (the largest fraction)."""
    f = peaks["sm_max_mhz"] * 1e6
    s = ms_per_batch * 1e-3
    a, h = units["aes_block"], units["sha1_compression"]
    alu_ops = w["aes_blocks"] * a["alu"] + w["sha1_compressions"] * h["alu"]
    lds_ops = w["aes_blocks"] * a["smem"]
    alu_peak = SM_COUNT * ALU_LANES_PER_CLK_SM * f / 1e12       # T lane-ops/s
    lds_peak = SM_COUNT * LDS_LANES_PER_CLK_SM * f / 1e12
    alu = {"achieved": alu_ops / s / 1e12, "peak": alu_peak, "unit": "Tops/s"}
    lds = {"achieved": lds_ops / s / 1e12, "peak": lds_peak, "unit": "Tlookups/s"}
    hbm = {"achieved": w["hbm_bytes"] / s / 1e9, "peak": peaks["hbm_gbs"], "unit": "GB/s"}
    for x in (alu, lds, hbm):
        x["frac"] = x["achieved"] / x["peak"]
    return {"alu": alu, "lds": lds, "hbm": hbm,
            "basis": (f"ALU pipe {ALU_LANES_PER_CLK_SM} lanes/clk/SM, LDS {LDS_LANES_PER_CLK_SM} "
                      f"lanes/clk/SM, x {SM_COUNT} SMs x {peaks['sm_max_mhz']:.0f} MHz; per unit "
                      f"(SASS, {units['source']}): AES block {a['alu']} ALU + {a['smem']} LDS, "
                      f"SHA-1 compression {h['alu']} ALU ({h['fma']} more on the FMA pipe); HBM "
                      f"D + 48 + C + 16 B per packet vs {peaks['source']} copy bandwidth")}


def load_traffic(kernel, cfg_name):
    """DRAM bytes per batch of `kernel` from the committed ncu summary, if any."""
    p = os.path.join(ROOT, "profiles", "ncu_kernels.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(f"{kernel}:{cfg_name}", {}).get("dram_bytes_per_launch")
    except Exception:
        return None


def pct(v, q):
    return float(np.percentile(np.asarray(v, np.float64), q)) if len(v) else None


def size_key(size):
    return str(size)


# --------------------------------------------------------------------------- ours
class Ctx:
    """Process-group / device plumbing of one rank."""

    def __init__(self, args):
        import torch
        import torch.distributed as dist
        self.torch, self.dist = torch, dist
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        self.local = int(os.environ.get("LOCAL_RANK", "0"))
        if self.world != args.gpus:
            raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={self.world}: launch one "
                             f"process per GPU (bench.py re-launches itself under torchrun when "
                             f"WORLD_SIZE is unset)")
        # BENCH_SHARE_GPU=1 (a plumbing check, not a measurement): every rank on
        # cuda:0 and gloo for the reductions, so the multi-rank flow (shards,
        # per-rank rings, barriers, max / sum over ranks) runs on a one-GPU box
        self.share = os.environ.get("BENCH_SHARE_GPU") == "1" and self.world > 1
        if self.share:
            self.local = 0
        torch.cuda.set_device(self.local)
        self.dev = torch.device("cuda", self.local)
        self.red_dev = torch.device("cpu") if self.share else self.dev
        if self.world > 1:
            if self.share:
                dist.init_process_group("gloo")
            else:
                dist.init_process_group("nccl", device_id=self.dev)
        self.peaks = load_peaks()
        self.l2 = int(getattr(torch.cuda.get_device_properties(self.dev), "L2_cache_size", 126 << 20))
        self.flush_buf = torch.empty(256 << 20, dtype=torch.uint8, device=self.dev)

    def barrier(self):
        if self.world > 1:
            if self.share:
                self.dist.barrier()
            else:
                self.dist.barrier(device_ids=[self.local])

    def flush(self):
        self.flush_buf.zero_()

    def max_ms(self, ms):
        return shard.max_over_ranks(ms, device=self.red_dev)

    def sum_all(self, d):
        return shard.reduce_counters(d, device=self.red_dev)


def measure_outbound(ctx, args, cfg_id, size, steps, warmup, full):
    """One workload (cfg_id / size) on this rank: the ring-timed headline pass,
    per-batch timestamps, and (full) the process_batch / graph / isolated
    comparisons and the profiled per-kernel pass."""
    torch = ctx.torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    p, b = shard.rank_workload(cfg_id, PKTS_PER_GPU, size, N_SA_TOTAL, ctx.rank, ctx.world)
    t = nba_ipsec.SATable(p, device=ctx.local, max_batch=PKTS_PER_GPU)
    if args.pipeline is not None:
        t.set_pipeline(args.pipeline)
    db = device.to_device(b, ctx.dev)
    R = int(os.environ.get("BENCH_NROT", 0)) or device.ring_slot_count(b.in_len, b.n, ctx.l2)
    dbs = [db] + [device.clone(db) for _ in range(R - 1)]
    slots = [(*d.args(), b.n) for d in dbs]
    ring = t.ring(slots)
    form = {0: "graph", 1: "persistent", 2: "pipelined", 3: "free", 4: "roles"}[ring.form]
    # settle clocks (>= 0.3 s of back-to-back batches), then >= W warm-up batches
    t_end = time.time() + 0.3
    while time.time() < t_end:
        ring.run_batches(4 * R)
        torch.cuda.synchronize()
    ring.run_batches(max(warmup, 2 * R))
    torch.cuda.synchronize()
    ctx.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(ctx.local) as clk:
        torch.cuda.synchronize()
        gpu_lead(torch)
        e0.record()
        ring.run_batches(steps)            # ALL K timed batches: ONE persistent launch
        e1.record()
        torch.cuda.synchronize()
    ctx.barrier()
    tot_ms = e0.elapsed_time(e1)
    res = {"b": b, "p": p, "R": R, "form": form, "tot_ms": tot_ms, "clk": clk, "launches": 1}
    # per-batch device timestamps (a second, identical pass)
    per_batch = None
    if ring.form != 0:
        ts = torch.zeros(steps + 1, dtype=torch.int64, device=ctx.dev)
        ring.set_timestamps(ts)
        ring.run_batches(steps)
        torch.cuda.synchronize()
        ring.set_timestamps(None)
        v = ts.cpu().numpy().astype(np.int64)
        d_us = np.diff(v)[1:] / 1e3         # batch 0 includes the ring's start-up
        per_batch = {"median_us": pct(d_us, 50), "p10_us": pct(d_us, 10), "p90_us": pct(d_us, 90),
                     "mean_us": float((v[-1] - v[1]) / 1e3 / max(steps - 1, 1)),
                     "first_us": float((v[1] - v[0]) / 1e3), "n": int(d_us.size)}
    res["per_batch"] = per_batch
    ring.close()
    if full:
        runs = [(lambda d=d: t.process(*d.args(), n=b.n)) for d in dbs]
        # (a) the same K batches as process_batch launches, back to back
        for k in range(2 * R):
            runs[k % R]()
        torch.cuda.synchronize()
        gpu_lead(torch)
        e0.record()
        for k in range(steps):
            runs[k % R]()
        e1.record()
        torch.cuda.synchronize()
        res["launch_loop_ms"] = e0.elapsed_time(e1)
        res["lpb"] = t.launches_per_batch()
        # (b) CUDA-graph replay of the slots' launches (the ring's graph form)
        os.environ["NBA_IPSEC_RING_GRAPH"] = "1"
        try:
            g = t.ring(slots)
        finally:
            del os.environ["NBA_IPSEC_RING_GRAPH"]
        g.run_batches(2 * R)
        torch.cuda.synchronize()
        gpu_lead(torch)
        e0.record()
        g.run_batches(steps)
        e1.record()
        torch.cuda.synchronize()
        res["graph_ms"] = e0.elapsed_time(e1)
        g.close()
        # (b') the software-pipelined ring form on the same slots (the default
        # before the role-split ring; set_form), when the ring's default is
        # another persistent form
        if form == "roles":
            pr = t.ring(slots)
            pr.set_form(nba_ipsec.Ring.PIPELINED)
            pr.run_batches(2 * R)
            torch.cuda.synchronize()
            gpu_lead(torch)
            e0.record()
            pr.run_batches(steps)
            e1.record()
            torch.cuda.synchronize()
            res["pipe_ring_ms"] = e0.elapsed_time(e1)
            pr.close()
        # (c) isolated batches: L2 flushed before each, one event pair per batch
        iso = min(steps, 50)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(iso)]
        for k in range(iso):
            ctx.flush()
            ev[k][0].record()
            runs[0]()
            ev[k][1].record()
        torch.cuda.synchronize()
        res["iso_ms"] = [a.elapsed_time(c) for a, c in ev]
    res["ctr"] = t.counters()
    t.close()
    del dbs
    return res


def rates(ctx, res, steps, ms=None):
    """Whole-job Gbps / Mpps / ESP-payload Gbps over all ranks for `steps`
    batches per rank in `ms` (default: the ring-timed pass), max over ranks."""
    b = res["b"]
    ms_max = ctx.max_ms(res["tot_ms"] if ms is None else ms)
    s = ms_max * 1e-3
    tot = ctx.sum_all({"pkts_ok": frame_bits(b) / 8.0, "pkts_dropped": 0, "bytes_in": b.n,
                       "bytes_out": int(b.in_len.astype(np.int64).sum()), "batches": 0})
    return {"gbps": 8.0 * tot["pkts_ok"] * steps / s / 1e9, "mpps": tot["bytes_in"] * steps / s / 1e6,
            "esp_payload_gbps": 8.0 * tot["bytes_out"] * steps / s / 1e9,
            "ms_per_step": ms_max / steps}


def measure_inbound(ctx, args, cfg_id, steps, warmup, form=None):
    """ESP inbound on the same traffic: the library's own outbound
    output of R consecutive batches of the config (> 2x L2 touched per
    rotation, every batch L2-cold), each in its own device buffers,
    decapsulated back to back, K batches between one CUDA event pair.  Sequence
    numbers grow along the rotation, so every packet is fresh and accepted;
    when the rotation wraps the receive windows are reset (one small kernel,
    inside the timed region).  The rotation runs through the inbound batch ring
    (nba_ipsec_ring_run_batches, one call per rotation)."""
    torch = ctx.torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    size = CFG_SIZE[cfg_id]
    p, b = shard.rank_workload(cfg_id, PKTS_PER_GPU, size, N_SA_TOTAL, ctx.rank, ctx.world)
    t_out = nba_ipsec.SATable(p, device=ctx.local, max_batch=PKTS_PER_GPU)
    db = device.to_device(b, ctx.dev)
    R = device.ring_slot_count(b.in_len, b.n, ctx.l2)
    esp = []
    for _ in range(R):
        ob, ol = torch.empty_like(db.out_buf), torch.zeros_like(db.out_len)
        t_out.process(db.in_buf, db.in_off, db.in_len, db.sa_idx, ob, db.out_off, ol, n=b.n)
        esp.append((ob, ol, torch.empty_like(db.out_buf), torch.zeros_like(db.out_len)))
    torch.cuda.synchronize()
    esp_len = esp[0][1][:b.n].cpu().numpy().view(np.uint16).astype(np.int64)
    t_out.close()
    t = nba_ipsec.SATable(p, device=ctx.local, max_batch=PKTS_PER_GPU)
    t.enable_inbound()
    if form is not None:             # force a form (default: the library's choice by length)
        os.environ["NBA_IPSEC_RING_IN_PIPE"] = "1" if form == "pipelined" else "0"
    try:
        ring = t.ring_inbound([(e[0], db.out_off, e[1], db.sa_idx, e[2], db.out_off, e[3], None, b.n)
                               for e in esp])
    finally:
        os.environ.pop("NBA_IPSEC_RING_IN_PIPE", None)

    def timed_batches(k_steps):
        left = k_steps
        while left:
            if ring.cursor == 0:
                t.reset_inbound()
            nb = min(left, R - ring.cursor)
            ring.run_batches(nb)
            left -= nb

    timed_batches(max(warmup, R))
    torch.cuda.synchronize()
    ctx.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gpu_lead(torch)
    e0.record()
    timed_batches(steps)
    e1.record()
    torch.cuda.synchronize()
    ctx.barrier()
    tot_ms = e0.elapsed_time(e1)
    ctr = t.in_counters()
    ok_all = ctr["pkts_ok"] == ctr["batches"] * b.n
    same = bool(torch.equal(esp[-1][3][:b.n].to(torch.int32), db.in_len[:b.n].to(torch.int32)))
    form = {0: "graph", 1: "persistent", 2: "pipelined", 3: "free", 4: "roles"}[ring.form]
    ring.close()
    del esp
    t.close()
    tot_max = ctx.max_ms(tot_ms)
    red = ctx.sum_all({"pkts_ok": frame_bits(b) / 8.0, "pkts_dropped": 0, "bytes_in": b.n,
                       "bytes_out": float((esp_len + 14).sum()), "batches": 0})
    sec = tot_max * 1e-3
    return {"gbps": 8.0 * red["pkts_ok"] * steps / sec / 1e9,
            "gbps_esp_wire": 8.0 * red["bytes_out"] * steps / sec / 1e9,
            "mpps": red["bytes_in"] * steps / sec / 1e6, "us_per_step": 1e3 * tot_max / steps,
            "all_accepted": bool(ok_all), "lengths_match_outbound_input": same, "ring_form": form}


def measure_flows(ctx, args, cfg_id, steps, warmup, n_flows=65536):
    """Flow -> SA lookup on the config's traffic rewritten to
    n_flows registered 5-tuples (5% unknown): the lookup kernel alone and the
    whole path taking its SAs from the flow table (sa_idx = NULL); and
    single-ingress dispatch into 8 owners' receive buffers (one GPU standing in
    for NVLink peers)."""
    torch = ctx.torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec, redistribute
    size = CFG_SIZE[cfg_id]
    p, b = shard.rank_workload(cfg_id, PKTS_PER_GPU, size, N_SA_TOTAL, ctx.rank, ctx.world)
    f = gen.make_flows(n_flows, len(p.spi), cfg_id=cfg_id, rank=ctx.rank)
    gen.apply_flows(b, f, cfg_id=cfg_id, miss=0.05)
    t = nba_ipsec.SATable(p, device=ctx.local, max_batch=PKTS_PER_GPU)
    t.set_flow_table(f)
    db = device.to_device(b, ctx.dev)
    sa_out = torch.empty(b.n, dtype=torch.int32, device=ctx.dev)
    cap_b = int(b.in_len.astype(np.int64).sum()) + 64
    rxs = [redistribute.alloc_rx(b.n, cap_b, ctx.dev) for _ in range(8)]
    table = redistribute.rx_table(rxs, ctx.dev)
    ws = torch.empty(nba_ipsec.route_workspace_bytes(b.n, 8), dtype=torch.uint8, device=ctx.dev)
    dcnt = torch.zeros(9, dtype=torch.int64, device=ctx.dev)
    dbyt = torch.zeros(9, dtype=torch.int64, device=ctx.dev)
    fns = {
        "lookup": lambda: t.lookup_sa(db.in_buf, db.in_off, db.in_len, sa_out, n=b.n),
        "path_with_lookup": lambda: t.process(db.in_buf, db.in_off, db.in_len, None, db.out_buf,
                                              db.out_off, db.out_len, n=b.n),
        "dispatch_8_owners": lambda: nba_ipsec.route_dispatch(
            db.in_buf, db.in_off, db.in_len, db.sa_idx, b.n, len(p.spi), None, 8, ws, table, b.n,
            cap_b, dcnt, dbyt),
    }
    out = {}
    for name, fn in fns.items():
        for _ in range(warmup):
            ctx.flush()
            fn()
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(steps)]
        for k in range(steps):
            ctx.flush()
            ev[k][0].record()
            fn()
            ev[k][1].record()
        torch.cuda.synchronize()
        ms = ctx.max_ms(sum(a.elapsed_time(c) for a, c in ev) / steps)
        out[name] = {"us": 1e3 * ms, "mpps": b.n / (ms * 1e-3) / 1e6}
    moved = 2 * int(b.in_len.astype(np.int64).sum()) + b.n * 28
    out["dispatch_8_owners"]["hbm_frac"] = moved / (out["dispatch_8_owners"]["us"] * 1e-6) / 1e9 / \
        ctx.peaks["hbm_gbs"]
    out["n_flows"], out["miss_fraction"] = n_flows, 0.05
    t.close()
    del rxs
    return out


def measure_alb(ctx, args, cfg_id, n_steps=1500, fixed_steps=20):
    """Adaptive split with two devices emulated on one GPU: device 0
    runs the fused path once per packet, device 1 twice (half the throughput),
    each with its own SA table holding every SA.  Every step routes one ingress
    batch of the config by the owner map (route_pack_map), then each device
    processes its share, timed alone with CUDA events on its own stream; the
    controller observes the max of the two (parallel devices).  Counters of SAs
    that change owner are handed over."""
    torch = ctx.torch
    from paper_conf_eurosys_kimjlmsm15_b200 import alb, device, nba_ipsec, redistribute
    size = CFG_SIZE[cfg_id]
    p, b = shard.rank_workload(cfg_id, PKTS_PER_GPU, size, N_SA_TOTAL, 0, 1, layout="packed")
    n_sa = len(p.spi)
    tabs = [nba_ipsec.SATable(p, device=ctx.local, max_batch=PKTS_PER_GPU) for _ in range(2)]
    scratch = nba_ipsec.SATable(p, device=ctx.local, max_batch=PKTS_PER_GPU)
    sts = [torch.cuda.Stream(device=ctx.dev) for _ in range(2)]
    db = device.to_device(b, ctx.dev)
    main = torch.cuda.current_stream()

    def step(sa_map_t):
        pk = redistribute.pack(db, b.n, n_sa, 2, sa_map=sa_map_t)
        dts = []
        for d in range(2):
            n, ioff, ilen, sa, ooff, olen, obuf = redistribute.local_views(pk, d)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            sts[d].wait_stream(main)
            with torch.cuda.stream(sts[d]):
                e0.record(sts[d])
                tabs[d].process(pk.buf, ioff, ilen, sa, obuf, ooff, olen, n=n, stream=sts[d])
                if d == 1:
                    scratch.process(pk.buf, ioff, ilen, sa, torch.empty_like(obuf), ooff,
                                    torch.empty_like(olen), n=n, stream=sts[d])
                e1.record(sts[d])
            e1.synchronize()
            dts.append(int(e0.elapsed_time(e1) * 1e6))
        main.wait_stream(sts[0])
        main.wait_stream(sts[1])
        return dts, pk.counts

    def map_tensor(sa_map):
        return torch.from_numpy(sa_map.view(np.int32)).to(ctx.dev)

    fixed = {}
    for k in (0, 4, 8, 12, 16, 25):
        _, m = nba_ipsec.alb_assign(n_sa, 2, [k], 25)
        mt = map_tensor(m)
        for _ in range(3):
            step(mt)
        ms = sum(max(step(mt)[0]) for _ in range(fixed_steps)) / fixed_steps / 1e6
        fixed[str(k / 25)] = round(b.n / (ms * 1e-3) / 1e6, 1)
    bal = alb.Balancer(n_sa, 2, history=64, update_ns=1_000_000)
    owner, sa_map = bal.assignment()
    mt = map_tensor(sa_map)
    t_ns, traj, tail, ho_us = 0, [int(bal.node_step[0])], [], []
    for j in range(n_steps):
        dts, counts = step(mt)
        t_ns += max(dts)
        if j >= n_steps - 200:
            tail.append(max(dts) / 1e6)
        if bal.observe(t_ns, dts, counts):
            new_owner, new_map = bal.assignment()
            h0 = time.perf_counter_ns()
            alb.handover_tables(tabs, owner, new_owner)
            ho_us.append((time.perf_counter_ns() - h0) / 1e3)
            owner, sa_map = new_owner, new_map
            mt = map_tensor(sa_map)
            traj.append(int(bal.node_step[0]))
    for t in tabs + [scratch]:
        t.close()
    ms_tail = float(np.mean(tail))
    best_w = max(fixed, key=fixed.get)
    mpps = b.n / (ms_tail * 1e-3) / 1e6
    return {"devices": "2 emulated on one B200 (device 1 does the work twice); step = max of the two",
            "workload": gen.CONFIGS[cfg_id]["name"], "updates": len(traj) - 1,
            "w_final": traj[-1] / 25, "w_last10_mean": float(np.mean(traj[-10:])) / 25,
            "mpps_last200": mpps, "mpps_fixed_w": fixed, "best_fixed_w": float(best_w),
            "alb_vs_best_fixed": mpps / fixed[best_w],
            "handover_us_mean": float(np.mean(ho_us)) if ho_us else None}


def run_e2e(ctx, args):
    """Same metric through nba_ipsec_process_batch_host: every step copies the
    step's inputs from pinned host memory and reads back the results."""
    torch = ctx.torch
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    size = CFG_SIZE[args.config]
    p, b = shard.rank_workload(args.config, PKTS_PER_GPU, size, N_SA_TOTAL, ctx.rank, ctx.world,
                               layout="packed", out_pad=53)
    t = nba_ipsec.SATable(p, device=ctx.local, max_batch=PKTS_PER_GPU)
    in_bytes = int(b.in_off[-1]) + int(b.in_len[-1])
    out_bytes = int(b.out_pool_bytes)
    t.reserve_host_io(in_bytes, out_bytes)
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()  # noqa: E731
    h_in = pin(b.in_buf)
    h_off, h_len, h_sa = pin(b.in_off.view(np.int32)), pin(b.in_len.view(np.int16)), pin(b.sa_idx.view(np.int32))
    h_ooff = pin(b.out_off.view(np.int32))
    h_out = torch.empty(out_bytes, dtype=torch.uint8).pin_memory()
    h_olen = torch.empty(b.n, dtype=torch.int16).pin_memory()
    st = torch.cuda.current_stream(ctx.dev)

    def step():
        t.process_host(h_in, h_off, h_len, h_sa, h_out, h_ooff, h_olen, in_bytes, out_bytes,
                       n=b.n, stream=st)

    for _ in range(max(3, args.warmup)):
        step()
    t.host_wait(st)
    torch.cuda.synchronize()
    ctx.barrier()
    steps = max(5, args.steps // 2)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gpu_lead(torch, 50.0)
    e0.record()
    for _ in range(steps):
        step()
    t.host_wait(st)            # the last step's outputs are in host memory
    e1.record()
    torch.cuda.synchronize()
    ctx.barrier()
    ms = ctx.max_ms(e0.elapsed_time(e1))
    tot = ctx.sum_all({"pkts_ok": frame_bits(b) / 8.0, "pkts_dropped": 0, "bytes_in": b.n,
                       "bytes_out": 0, "batches": 0})
    t.close()
    h2d = in_bytes + b.n * (4 + 2 + 4 + 4)
    d2h = out_bytes + b.n * 2
    return {"value": 8.0 * tot["pkts_ok"] * steps / (ms * 1e-3) / 1e9, "unit": "Gbps",
            "mpps": tot["bytes_in"] * steps / (ms * 1e-3) / 1e6,
            "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
            "steps": steps, "ms_per_step": ms / steps,
            "api": "nba_ipsec_process_batch_host (pinned host buffers: packed datagrams H2D by copy, "
                   "per-packet metadata read and out_len written in place over PCIe by the kernels, "
                   "output pool D2H by copy, every step; 2 staging slots pipelined)"}


def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


def oracle_leg(p, b, threads, budget_s):
    """The oracle as it stands (plain C -O2, SAs partitioned s mod T over T
    threads) on a bounded sample of batch b: the first m packets, m sized from a
    probe so one call takes ~budget_s / 3, repeated until budget_s."""
    import oracle
    sas = oracle.make_sas(p)
    n_sa = len(p.spi)
    out = np.zeros(b.out_pool_bytes, np.uint8)

    def sub(m):
        return gen.Batch(n=m, in_buf=b.in_buf, in_off=b.in_off[:m], in_len=b.in_len[:m],
                         sa_idx=b.sa_idx[:m], out_off=b.out_off[:m], out_pool_bytes=b.out_pool_bytes,
                         frame_len=b.frame_len[:m])
    probe = sub(min(b.n, 2048))
    t0 = time.perf_counter()
    oracle.process_batch(sas, n_sa, probe, n_threads=threads, out_buf=out)
    per_pkt = (time.perf_counter() - t0) / probe.n
    m = int(max(256, min(b.n, budget_s / 3.0 / max(per_pkt, 1e-9))))
    sb = sub(m)
    reps, t0 = 0, time.perf_counter()
    while True:
        oracle.process_batch(sas, n_sa, sb, n_threads=threads, out_buf=out)
        reps += 1
        el = time.perf_counter() - t0
        if el >= budget_s:
            break
    return {"gbps": frame_bits(sb) * reps / el / 1e9, "mpps": m * reps / el / 1e6, "threads": threads,
            "sample": f"first {m} of {b.n} packets x {reps} ({el:.1f} s)"}


def cpu_baselines(budget_s):
    """SURVEY §8(d) oracle timing: configs[0] in ms (1 thread), and configs[1..3]
    on 1 thread and on all host threads (bounded samples)."""
    import oracle
    T = len(os.sched_getaffinity(0))
    c = gen.CONFIGS[1]
    p1 = gen.make_sas(c["n_sa"], cfg_id=1)
    b1 = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=1)
    ms = []
    t_end = time.perf_counter() + 0.5
    while time.perf_counter() < t_end or len(ms) < 5:
        sas = oracle.make_sas(p1)
        t0 = time.perf_counter()
        oracle.process_batch(sas, 1, b1, n_threads=1)
        ms.append((time.perf_counter() - t0) * 1e3)
    legs = {"c1_64x64B_1sa_ms_1thread": float(np.median(ms))}
    for cfg in (2, 3, 4):
        p, b = shard.rank_workload(cfg, PKTS_PER_GPU, CFG_SIZE[cfg], N_SA_TOTAL, 0, 1)
        name = gen.CONFIGS[cfg]["name"]
        legs[name] = {"1": oracle_leg(p, b, 1, budget_s), str(T): oracle_leg(p, b, T, budget_s)}
    return {"cpu_model": cpu_model(), "threads_available": T, "legs": legs}


def run_ours(args):
    ctx = Ctx(args)
    torch = ctx.torch
    units = sass_units()
    main_cfg = args.config
    steps, warmup = args.steps, args.warmup
    head = measure_outbound(ctx, args, main_cfg, CFG_SIZE[main_cfg], steps, warmup, full=True)
    agg = rates(ctx, head, steps)
    w = work_model(head["b"])
    ms_batch = agg["ms_per_step"]
    roof = roofline(ms_batch, w, ctx.peaks, units)
    kname = {"graph": "fused", "roles": "fused_ring_roles"}.get(head["form"], "fused_ring")
    roof_line = {"kernel": {"pipelined": "k_fused_ring_pipe", "roles": "k_fused_ring_roles",
                            "free": "k_fused_ring_free"}.get(head["form"], "k_fused_ring"),
                 "bound": "alu", "achieved": roof["alu"]["achieved"], "peak": roof["alu"]["peak"],
                 "unit": "Tops/s", "frac": roof["alu"]["frac"],
                 "traffic": load_traffic(kname, gen.CONFIGS[main_cfg]["name"]),
                 "traffic_algorithmic": w["hbm_bytes"],
                 "lds_frac": roof["lds"]["frac"], "hbm_frac": roof["hbm"]["frac"],
                 "basis": roof["basis"]}
    # ---- configs[4] sweep (and configs[2], configs[3]) ------------------------
    by_size = {size_key(CFG_SIZE[main_cfg]): {"gbps": agg["gbps"], "mpps": agg["mpps"],
                                             "us": 1e3 * agg["ms_per_step"],
                                             "esp_payload_gbps": agg["esp_payload_gbps"],
                                             "alu_frac": roof["alu"]["frac"],
                                             "p50_us": (head["per_batch"] or {}).get("median_us")}}
    sweep_detail = {}
    if not args.no_sweep:
        k_sw = max(20, min(steps, 100))
        for cfg_id, size in SWEEP:
            if size == CFG_SIZE[main_cfg]:
                continue
            r = measure_outbound(ctx, args, cfg_id, size, k_sw, max(3, warmup // 2), full=False)
            a = rates(ctx, r, k_sw)
            rf = roofline(a["ms_per_step"], work_model(r["b"]), ctx.peaks, units)
            by_size[size_key(size)] = {"gbps": a["gbps"], "mpps": a["mpps"],
                                       "us": 1e3 * a["ms_per_step"],
                                       "esp_payload_gbps": a["esp_payload_gbps"],
                                       "alu_frac": rf["alu"]["frac"], "lds_frac": rf["lds"]["frac"],
                                       "hbm_frac": rf["hbm"]["frac"],
                                       "p50_us": (r["per_batch"] or {}).get("median_us")}
            sweep_detail[size_key(size)] = {"per_batch": r["per_batch"], "ring_slots": r["R"],
                                            "form": r["form"], "steps": k_sw}
    # ---- ESP inbound (f2), flow lookup / dispatch (f3), adaptive split (f4) -----
    inbound = {}
    if not args.no_inbound:
        for cfg_id in (2, 3, 4):
            inbound[size_key(CFG_SIZE[cfg_id])] = measure_inbound(ctx, args, cfg_id,
                                                                 max(10, steps // 4),
                                                                 max(3, warmup // 2))
        # the other form at 64 B on the same traffic: the CUDA-graph ring of
        # one-kernel launches (the library picks the pipelined ring there)
        inbound["64_graph_ring"] = measure_inbound(ctx, args, 2, max(10, steps // 4),
                                                   max(3, warmup // 2), form="graph")
    flows = None
    if not args.no_inbound:
        flows = measure_flows(ctx, args, main_cfg, max(10, steps // 4), max(3, warmup // 2))
    alb_res = None
    if ctx.world == 1 and not args.no_alb:
        alb_res = measure_alb(ctx, args, 3)
    e2e = run_e2e(ctx, args)
    cpu = None
    if ctx.rank == 0 and ctx.world == 1 and not args.no_cpu:
        cpu = cpu_baselines(args.cpu_seconds)
    ctr_all = ctx.sum_all(head["ctr"])
    launch_ms = ctx.max_ms(head.get("launch_loop_ms", 0.0))
    graph_ms = ctx.max_ms(head.get("graph_ms", 0.0))
    pipe_ms = ctx.max_ms(head.get("pipe_ring_ms", 0.0))
    if ctx.rank == 0:
        clk = head["clk"].summary()
        nm = gen.CONFIGS[main_cfg]["name"]
        T = (cpu or {}).get("threads_available")
        leg = (cpu or {}).get("legs", {}).get(nm, {})
        cpu_line = None
        if cpu:
            allc = leg[str(T)]
            cpu_line = {"value": allc["gbps"], "unit": "Gbps", "cores": T, "kind": "oracle",
                        "sample": f"{nm}: {allc['sample']} on {T} threads", "mpps": allc["mpps"],
                        "one_thread_gbps": leg["1"]["gbps"], "cpu_model": cpu["cpu_model"],
                        "c1_64x64B_1sa_ms_1thread": cpu["legs"]["c1_64x64B_1sa_ms_1thread"]}
        pb = head["per_batch"] or {}
        out = {
            "metric": METRIC,
            "value": agg["gbps"],
            "unit": "Gbps",
            "mpps": agg["mpps"],
            "n_gpus": ctx.world,
            "steps": steps,
            "warmup": warmup,
            "ms_per_step": agg["ms_per_step"],
            "higher_is_better": True,
            "scaling": "weak",
            "vs_baseline": None,
            "dtype": "u8",
            "data": "synthetic (seeded random IPv4/UDP, random SA keys; PAPER.md:395 workload shape)",
            "config": {"workload": f"configs[{main_cfg - 1}]: {nm}", "frame_bytes": CFG_SIZE[main_cfg],
                       "packets_per_gpu": PKTS_PER_GPU, "n_sa_total": N_SA_TOTAL,
                       "global_batch": PKTS_PER_GPU * ctx.world,
                       "parallelism": f"sa-hash shard x{ctx.world} (no data-path collective)"
                                      + (" -- BENCH_SHARE_GPU: every rank on cuda:0 with gloo "
                                         "reductions, a plumbing check, not a measurement"
                                         if ctx.share else ""),
                       "l2": f"inputs larger than L2: batches rotate over {head['R']} device copies "
                             "(> 2x L2 touched per rotation), SA table resident",
                       "timing": f"all {steps} timed batches in ONE nba_ipsec_ring_run_batches call "
                                 f"({head['form']} persistent ring, 1 launch, its start-up included) "
                                 "between one CUDA event pair, barrier + sync both sides, max over "
                                 "ranks; a sleep kernel ahead of the start event keeps host enqueue "
                                 "latency out of the device time"},
            "roofline": roof_line,
            "gbps_by_size": {k: round(v["gbps"], 1) for k, v in by_size.items()},
            "us_by_size": {k: round(v["us"], 2) for k, v in by_size.items()},
            "esp_payload_gbps": agg["esp_payload_gbps"],
            "per_batch_us": {k: (round(v, 3) if isinstance(v, float) else v) for k, v in pb.items()},
            "cpu_baseline": cpu_line,
            "e2e": e2e,
            "gpu_launches": head["launches"],
            "clocks": clk,
            "compare": {"process_batch_loop_us": 1e3 * launch_ms / steps,
                        "graph_replay_us": 1e3 * graph_ms / steps,
                        "pipelined_ring_us": (1e3 * pipe_ms / steps) if pipe_ms else None,
                        "isolated_batch_us_mean": 1e3 * float(np.mean(head["iso_ms"])),
                        "ring_us": 1e3 * agg["ms_per_step"],
                        "launches_per_batch_unringed": head.get("lpb")},
            "by_size": by_size,
            "sweep": sweep_detail,
            "work_per_step_per_gpu": w,
            "cpu_legs": cpu,
            "counters": ctr_all,
            "inbound": inbound or None,
            "flow_lookup": flows,
            "adaptive_split": alb_res,
            # compact recap at the end of the line (kept in the driver's tail)
            "summary": {"Gbps": {k: round(v["gbps"], 1) for k, v in by_size.items()},
                        "us": {k: round(v["us"], 2) for k, v in by_size.items()},
                        "alu_frac": {k: round(v["alu_frac"], 3) for k, v in by_size.items()},
                        "inbound_Gbps": {k: round(v["gbps"], 1) for k, v in inbound.items()},
                        "p50_p10_p90_us": [pb.get("median_us"), pb.get("p10_us"), pb.get("p90_us")],
                        "oracle_Gbps_1t_Nt": [leg.get("1", {}).get("gbps"),
                                              leg.get(str(T), {}).get("gbps")] if cpu else None,
                        "n_gpus": ctx.world},
        }
        print(json.dumps(out), flush=True)
    if ctx.world > 1:
        ctx.dist.destroy_process_group()


# --------------------------------------------------------------------------- reference arm
def run_reference(args):
    """The oracle (this tier's reference arm) on the host cores, same metric and
    config as our arm.  Under torchrun only rank 0 works; others exit 0."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    size = CFG_SIZE[args.config]
    p, b = shard.rank_workload(args.config, PKTS_PER_GPU, size, N_SA_TOTAL, 0, 1)
    T = len(os.sched_getaffinity(0))
    sas = oracle.make_sas(p)
    out = np.zeros(b.out_pool_bytes, np.uint8)
    # bounded sample per step: as many packets as ~0.5 s of all-core work
    probe = min(b.n, 4096)
    sub = gen.Batch(n=probe, in_buf=b.in_buf, in_off=b.in_off[:probe], in_len=b.in_len[:probe],
                    sa_idx=b.sa_idx[:probe], out_off=b.out_off[:probe],
                    out_pool_bytes=b.out_pool_bytes, frame_len=b.frame_len[:probe])
    t0 = time.perf_counter()
    oracle.process_batch(sas, len(p.spi), sub, n_threads=T, out_buf=out)
    per_pkt = (time.perf_counter() - t0) / probe
    m = int(max(1024, min(b.n, 0.5 / max(per_pkt, 1e-9))))
    sb = gen.Batch(n=m, in_buf=b.in_buf, in_off=b.in_off[:m], in_len=b.in_len[:m],
                   sa_idx=b.sa_idx[:m], out_off=b.out_off[:m], out_pool_bytes=b.out_pool_bytes,
                   frame_len=b.frame_len[:m])
    for _ in range(args.warmup):
        oracle.process_batch(sas, len(p.spi), sb, n_threads=T, out_buf=out)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.process_batch(sas, len(p.spi), sb, n_threads=T, out_buf=out)
    el = time.perf_counter() - t0
    gbps = frame_bits(sb) * args.steps / el / 1e9
    line = {
        "impl": "reference",
        "metric": METRIC, "value": gbps, "unit": "Gbps", "mpps": m * args.steps / el / 1e6,
        "n_gpus": int(os.environ.get("WORLD_SIZE", "1")), "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": el * 1e3 / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": f"configs[{args.config - 1}]: {gen.CONFIGS[args.config]['name']}",
                   "frame_bytes": CFG_SIZE[args.config], "packets_per_gpu": PKTS_PER_GPU,
                   "n_sa_total": N_SA_TOTAL},
        "cpu_baseline": {"value": gbps, "unit": "Gbps", "cores": T, "kind": "oracle",
                         "sample": f"first {m} packets of the {b.n}-packet batch per step "
                                   f"(~0.5 s all-core work), {args.steps} steps",
                         "cpu_model": cpu_model()},
        "e2e": {"value": gbps, "unit": "Gbps", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def relaunch_under_torchrun(args):
    """--gpus N > 1 without a torchrun environment: exec torchrun with one
    process per GPU (NCCL communicator init printed, NCCL_DEBUG=INFO)."""
    import socket
    try:
        import torch
        have = torch.cuda.device_count()
    except Exception:
        have = 0
    if have < args.gpus and os.environ.get("BENCH_SHARE_GPU") != "1":
        raise SystemExit(f"bench.py: --gpus {args.gpus} requested but {have} CUDA device(s) visible")
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr", "127.0.0.1", "--master-port", str(port),
           os.path.abspath(__file__), *sys.argv[1:]]
    os.execvpe(cmd[0], cmd, env)


def parse_args(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--config", type=int, default=2, choices=[2, 3, 4])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--pipeline", type=int, default=None, help="0 fused, 1 unfused")
    ap.add_argument("--no-sweep", action="store_true")
    ap.add_argument("--no-inbound", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-alb", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=2.0,
                    help="per oracle leg (configs[1..3] x {1, N} threads)")
    args = ap.parse_args(argv)
    if args.warmup < 3:
        args.warmup = 3
    return args


def main():
    args = parse_args()
    if args.impl == "reference":
        run_reference(args)
        return
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        relaunch_under_torchrun(args)
    if int(os.environ.get("WORLD_SIZE", "1")) > 1:
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    run_ours(args)


if __name__ == "__main__":
    main()
