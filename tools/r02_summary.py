#!/usr/bin/env python
"""Summarise an r02 GPU session into profiles/ (committed evidence).

    python tools/r02_summary.py TAG

Reads gpurun_out/prof_TAG_ring_c{2,3,4}.ncu-rep (the ring's default form for the
config -- k_fused_ring_roles or k_fused_ring_pipe -- one run of 6 batch slots =
6 batches), gpurun_out/prof_TAG_in_c{2,3,4}.ncu-rep (inbound
one-kernel launch), gpurun_out/TAG_launches.csv (ncu launch list of
`bench.py --steps 22`), gpurun_out/microbench_TAG.json and
gpurun_out/bench_TAG.json; writes profiles/TAG_ncu_summary.md and updates
profiles/ncu_kernels.json (DRAM bytes per batch, read by bench.py as
roofline.traffic)."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
CFG = {2: "c2_64B_1024sa", 3: "c3_1514B_1024sa", 4: "c4_imix_1024sa"}
METRICS = [("gpu__time_duration.sum", "us", 1e-3, "us"),
           ("dram__bytes_read.sum", "DRAM rd MB", 1e-6, "byte"),
           ("dram__bytes_write.sum", "DRAM wr MB", 1e-6, "byte"),
           ("sm__inst_issued.avg.pct_of_peak_sustained_active", "issue %", 1, None),
           ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "ALU %", 1, None),
           ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA %", 1, None),
           ("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed", "L1 data pipe %", 1, None),
           ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem wavefronts", 1, None),
           ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "bank conflicts", 1, None),
           ("smsp__inst_executed.sum", "warp inst", 1, None),
           ("launch__registers_per_thread", "regs", 1, None)]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1e3, "msecond": 1e6, "ms": 1e6,
         "nsecond": 1, "us": 1e3}


def raw(rep):
    r = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True)
    rows = list(csv.reader(io.StringIO(r.stdout)))
    if len(rows) < 3:
        return None
    h, u, d = rows[0], rows[1], rows[2]
    out = {}
    if "Kernel Name" in h:
        k = d[h.index("Kernel Name")]
        out["kernel"] = k.split("(")[0].replace("nba::", "").replace("void ", "")
    for name, label, mul, kind in METRICS:
        if name in h:
            i = h.index(name)
            v = float(d[i].replace(",", "") or 0)
            if kind == "byte":
                v = v * SCALE.get(u[i], 1) * mul
            elif kind == "us":
                v = v * SCALE.get(u[i], 1) * mul        # -> ns * 1e-3 = us
            out[label] = v
    return out


def main():
    tag = sys.argv[1]
    lines = [f"# ncu summary, round tag `{tag}`", "",
             "Captured with `ncu --set full --clock-control none --import-source on` under gpurun "
             "(`tools/r02_final.sh`); serialised, cold-cache replays: times under ncu are not bench "
             "values, compare shares.  Ring rows: one launch of the ring's default form (kernel "
             "column) over a 6-slot ring (6 batches), per-batch figures = launch / 6.", ""]
    kj_path = os.path.join(PROF, "ncu_kernels.json")
    kj = json.load(open(kj_path)) if os.path.exists(kj_path) else {}
    for kind, title, div in (("ring", "batch ring, default form (per batch)", 6.0),
                             ("in", "ESP inbound, one-kernel launch", 1.0)):
        lines += [f"## {title}", "",
                  "| config | kernel | " + " | ".join(m[1] for m in METRICS) + " |",
                  "|---|---|" + "---|" * len(METRICS)]
        for c, name in CFG.items():
            rep = os.path.join(OUT, f"prof_{tag}_{kind}_c{c}.ncu-rep")
            if not os.path.exists(rep):
                continue
            v = raw(rep)
            if not v:
                continue
            cells = []
            for _, label, _, k in METRICS:
                x = v.get(label)
                if x is None:
                    cells.append("-")
                    continue
                if label in ("us", "DRAM rd MB", "DRAM wr MB", "warp inst", "smem wavefronts",
                             "bank conflicts"):
                    x = x / div
                cells.append(f"{x:.4g}")
            kern = v.get("kernel", "")
            lines.append(f"| {name} | {kern} | " + " | ".join(cells) + " |")
            key = ("in_fused" if kind != "ring" else
                   "fused_ring_roles" if "roles" in kern else "fused_ring") + ":" + name
            kj[key] = {"dram_bytes_per_launch": (v["DRAM rd MB"] + v["DRAM wr MB"]) * 1e6 / div,
                       "ncu_duration_us": v["us"] / div,
                       "note": "per batch of a 6-batch ring run" if kind == "ring" else "per launch",
                       "source": os.path.basename(rep)}
        lines.append("")
    kj["_round"] = tag
    json.dump(kj, open(kj_path, "w"), indent=1, sort_keys=True)
    lp = os.path.join(OUT, f"{tag}_launches.csv")
    if os.path.exists(lp):
        txt = open(lp).read()
        rows = [r for r in csv.reader(io.StringIO(txt[txt.find('"ID"'):])) if r]
        if rows:
            h = rows[0]
            ki, vi = h.index("Kernel Name"), h.index("Metric Value")
            agg = {}
            for r in rows[1:]:
                if len(r) > vi and r[vi].replace(",", "").replace(".", "").isdigit():
                    agg.setdefault(r[ki][:60], []).append(float(r[vi].replace(",", "")))
            tot = sum(sum(x) for k, x in agg.items() if "nba::" in k) or 1.0
            lines += ["## launch list (`bench.py --steps 22 --warmup 3 --no-sweep ...`, "
                      "`--metrics gpu__time_duration.sum`)", "",
                      "| kernel | launches | mean ns | share of our kernels |", "|---|---|---|---|"]
            for k, x in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
                share = 100.0 * sum(x) / tot if "nba::" in k else 0.0
                lines.append(f"| {k} | {len(x)} | {sum(x) / len(x):.0f} | {share:.1f}% |")
            lines.append("")
    mp = os.path.join(OUT, f"microbench_{tag}.json")
    if os.path.exists(mp):
        lines += ["## integer / shared-memory microbenchmarks (tools/microbench.cu)", "", "```",
                  open(mp).read().strip(), "```", ""]
    bp = os.path.join(OUT, f"bench_{tag}.json")
    if os.path.exists(bp):
        d = json.loads(open(bp).read().strip().split("\n")[-1])
        lines += ["## bench line (key fields)", "", "```",
                  json.dumps({k: d.get(k) for k in ("value", "ms_per_step", "gbps_by_size", "us_by_size",
                                                     "per_batch_us", "roofline", "compare", "clocks",
                                                     "gpu_launches")}, indent=1), "```", ""]
    open(os.path.join(PROF, f"{tag}_ncu_summary.md"), "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
