"""Summarise a gpurun round's ncu captures into profiles/ (committed).

    python tools/summarize_profiles.py TAG

Reads gpurun_out/prof_TAG_c{2,3,4}.ncu-rep (fused pipeline),
gpurun_out/prof_TAG_unfused_c3.ncu-rep, gpurun_out/launches_TAG.csv,
gpurun_out/microbench_TAG.json and gpurun_out/bench_TAG.json, and writes
profiles/TAG_ncu_summary.md and profiles/ncu_kernels.json (per-launch DRAM
bytes per kernel and config, used by bench.py as roofline.traffic).
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
CFG = {"c2": "c2_64B_1024sa", "c3": "c3_1514B_1024sa", "c4": "c4_imix_1024sa"}
METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("lts__t_bytes.sum", "l2_bytes"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_throughput_pct"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_active_pct"),
    ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "alu_pipe_pct"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "fma_pipe_pct"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "lsu_inst_pct"),
    ("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed", "l1_data_pipe_pct"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "shared_wavefronts"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "shared_bank_conflicts"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps_active_pct"),
    ("smsp__inst_executed.sum", "warp_instructions"),
    ("launch__registers_per_thread", "registers"),
    ("launch__block_size", "block"),
    ("launch__grid_size", "grid"),
    ("sm__cycles_elapsed.avg.per_second", "sm_clock"),
]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6,
         "usecond": 1e-6, "msecond": 1e-3, "nsecond": 1e-9, "Ghz": 1e9, "Mhz": 1e6}


ALIAS = {"aes": "aes_ctr", "hmac": "hmac_sha1"}


def short_name(full):
    """'void nba::k_fused<1>(nba::DevTable, ...)' -> 'fused' (bench.py's kernel names)."""
    n = full.split("(")[0].replace("void ", "").replace("nba::", "").split("<")[0]
    n = n[2:] if n.startswith("k_") else n
    return ALIAS.get(n, n)


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    h, units, data = rows[0], rows[1], rows[2:]
    res = []
    for r in data:
        d = {"kernel": short_name(r[h.index("Kernel Name")])}
        for m, short in METRICS:
            if m in h:
                v, u = r[h.index(m)].replace(",", ""), units[h.index(m)]
                try:
                    d[short] = float(v) * SCALE.get(u, 1.0)
                except ValueError:
                    d[short] = v
        res.append(d)
    return res


def main(tag):
    os.makedirs(PROF, exist_ok=True)
    lines = [f"# ncu summary, round tag `{tag}`", "",
             "Captured with `ncu --set full --clock-control none --import-source on` under gpurun "
             "(tools/gpu_round.sh); per launch, serialised and cold-cache.  Times under ncu are "
             "not bench values.", ""]
    kj = {}
    for c, name in CFG.items():
        rep = os.path.join(OUT, f"prof_{tag}_{c}.ncu-rep")
        if not os.path.exists(rep):
            continue
        rows = raw(rep)
        agg = collections.defaultdict(list)
        for d in rows:
            agg[d["kernel"]].append(d)
        lines += [f"## {name} (fused pipeline)", "",
                  "| kernel | us | DRAM rd MB | DRAM wr MB | issue % | ALU % | FMA % | LSU % | L1 data pipe % | smem wavefronts | bank conflicts | warp inst | regs |",
                  "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
        for k, ds in agg.items():
            d = collections.defaultdict(lambda: float("nan"))
            d.update({m: (v if isinstance(v, float) else float("nan")) for m, v in ds[-1].items()
                      if m != "kernel"})
            lines.append(
                f"| {k} | {d['duration'] * 1e6:.1f} | {d['dram_read'] / 1e6:.2f} | {d['dram_write'] / 1e6:.2f} | "
                f"{d['issue_active_pct']:.1f} | {d['alu_pipe_pct']:.1f} | {d['fma_pipe_pct']:.1f} | "
                f"{d['lsu_inst_pct']:.1f} | {d['l1_data_pipe_pct']:.1f} | {d['shared_wavefronts']:.3g} | "
                f"{d['shared_bank_conflicts']:.3g} | {d['warp_instructions']:.3g} | {d['registers']:.0f} |")
            kj[f"{k}:{name}"] = {"dram_bytes_per_launch": d["dram_read"] + d["dram_write"],
                                 "ncu_duration_us": d["duration"] * 1e6,
                                 "source": os.path.basename(rep)}
        lines.append("")
    for c, name in CFG.items():
        rep = os.path.join(OUT, f"prof_{tag}_ring_{c}.ncu-rep")
        if not os.path.exists(rep):
            continue
        lines += [f"## {name} batch ring (k_fused_ring: ONE launch walks a run of 4 batches; "
                  "per-batch figures = launch / 4)", "",
                  "| kernel | us / batch | DRAM rd MB / batch | DRAM wr MB / batch | issue % | ALU % | FMA % | LSU % | L1 data pipe % | warp inst / batch | regs |",
                  "|---|---|---|---|---|---|---|---|---|---|---|"]
        for d0 in raw(rep):
            d = collections.defaultdict(lambda: float("nan"))
            d.update({m: (v if isinstance(v, float) else float("nan")) for m, v in d0.items()})
            lines.append(f"| {d0['kernel']} | {d['duration'] * 1e6 / 4:.1f} | {d['dram_read'] / 4e6:.2f} | "
                         f"{d['dram_write'] / 4e6:.2f} | {d['issue_active_pct']:.1f} | "
                         f"{d['alu_pipe_pct']:.1f} | {d['fma_pipe_pct']:.1f} | {d['lsu_inst_pct']:.1f} | "
                         f"{d['l1_data_pipe_pct']:.1f} | {d['warp_instructions'] / 4:.3g} | {d['registers']:.0f} |")
            kj[f"fused_ring:{name}"] = {"dram_bytes_per_launch": (d["dram_read"] + d["dram_write"]) / 4,
                                        "ncu_duration_us": d["duration"] * 1e6 / 4,
                                        "note": "per batch of a 4-batch ring run",
                                        "source": os.path.basename(rep)}
        lines.append("")
    for c, name in CFG.items():
        rep = os.path.join(OUT, f"prof_{tag}_in_{c}.ncu-rep")
        if not os.path.exists(rep):
            continue
        lines += [f"## {name} ESP inbound (one kernel: k_in_fused<true>, replay decision inside)", "",
                  "| kernel | us | DRAM rd MB | DRAM wr MB | issue % | ALU % | LSU % | L1 data pipe % | warp inst | regs |",
                  "|---|---|---|---|---|---|---|---|---|---|"]
        for d0 in raw(rep):
            d = collections.defaultdict(lambda: float("nan"))
            d.update({m: (v if isinstance(v, float) else float("nan")) for m, v in d0.items()})
            lines.append(f"| {d0['kernel']} | {d['duration'] * 1e6:.1f} | {d['dram_read'] / 1e6:.2f} | "
                         f"{d['dram_write'] / 1e6:.2f} | {d['issue_active_pct']:.1f} | "
                         f"{d['alu_pipe_pct']:.1f} | {d['lsu_inst_pct']:.1f} | {d['l1_data_pipe_pct']:.1f} | "
                         f"{d['warp_instructions']:.3g} | {d['registers']:.0f} |")
            kj[f"{d0['kernel']}:{name}"] = {"dram_bytes_per_launch": d["dram_read"] + d["dram_write"],
                                            "ncu_duration_us": d["duration"] * 1e6,
                                            "source": os.path.basename(rep)}
        lines.append("")
    rep = os.path.join(OUT, f"prof_{tag}_unfused_c3.ncu-rep")
    if os.path.exists(rep):
        lines += ["## c3_1514B_1024sa (unfused ablation: gather / AES / HMAC / scatter)", "",
                  "| kernel | us | DRAM rd MB | DRAM wr MB | issue % | ALU % | LSU % | bank conflicts |",
                  "|---|---|---|---|---|---|---|---|"]
        for d0 in raw(rep):
            d = collections.defaultdict(lambda: float("nan"))
            d.update({m: (v if isinstance(v, float) else float("nan")) for m, v in d0.items()})
            d["kernel"] = d0["kernel"]
            lines.append(f"| {d['kernel']} | {d['duration'] * 1e6:.1f} | {d['dram_read'] / 1e6:.2f} | "
                         f"{d['dram_write'] / 1e6:.2f} | {d['issue_active_pct']:.1f} | "
                         f"{d['alu_pipe_pct']:.1f} | {d['lsu_inst_pct']:.1f} | {d['shared_bank_conflicts']:.3g} |")
            kj[f"{d['kernel']}:c3_1514B_1024sa:unfused"] = {
                "dram_bytes_per_launch": d["dram_read"] + d["dram_write"],
                "ncu_duration_us": d["duration"] * 1e6}
        lines.append("")
    lc = os.path.join(OUT, f"launches_{tag}.csv")
    if os.path.exists(lc):
        rows = list(csv.reader(open(lc)))
        hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        h = rows[hdr]
        ki, vi = h.index("Kernel Name"), h.index("Metric Value")
        agg = collections.defaultdict(list)
        for r in rows[hdr + 1:]:
            if len(r) > vi:
                agg[r[ki].split("(")[0].replace("void ", "")].append(float(r[vi].replace(",", "")))
        tot = sum(sum(v) for k, v in agg.items() if k.startswith("nba::"))
        lines += ["## launch list (bench.py --steps 5, `--metrics gpu__time_duration.sum`)", "",
                  "| kernel | launches | mean ns | share of our kernels |", "|---|---|---|---|"]
        for k, v in agg.items():
            share = sum(v) / tot if k.startswith("nba::") and tot else 0
            lines.append(f"| {k[:60]} | {len(v)} | {sum(v) / len(v):.0f} | {share * 100:.1f}% |")
        lines.append("")
    mb = os.path.join(OUT, f"microbench_{tag}.json")
    if os.path.exists(mb):
        lines += ["## integer / shared-memory microbenchmarks (tools/microbench.cu)", "", "```",
                  open(mb).read().strip(), "```", ""]
    bj = os.path.join(OUT, f"bench_{tag}.json")
    if os.path.exists(bj):
        try:
            b = json.load(open(bj))
            lines += ["## bench.py line", "", "```", json.dumps(b, indent=1)[:6000], "```", ""]
        except Exception:
            pass
    with open(os.path.join(PROF, f"{tag}_ncu_summary.md"), "w") as f:
        f.write("\n".join(lines))
    old = {"_round": tag}
    pj = os.path.join(PROF, "ncu_kernels.json")
    old.update(kj)
    with open(pj, "w") as f:
        json.dump(old, f, indent=1)
    print("\n".join(lines[:80]))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r01")
