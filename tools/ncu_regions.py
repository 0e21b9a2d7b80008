#!/usr/bin/env python
"""Warp-stall samples and executed instructions of an ncu capture, by source
function (the SASS of the kernel attributed with nvdisasm -gi line info, as in
tools/sass_hist.py).

    ncu -i prof.ncu-rep --page source --csv --print-source sass > src.csv
    python tools/ncu_regions.py src.csv [--kernel k_fused_ring_pipe]

Prints, per region: share of stall samples, executed warp instructions and the
top stall reasons -- where the time of the kernel goes."""
import argparse
import collections
import csv
import os
import re
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import sass_hist  # noqa: E402

REGIONS = [  # (name, file, function) innermost match wins, in this order
    ("sha1", "sha1.cuh", "sha1_compress_fma"),
    ("aes_step", "fused_common.cuh", "aes4_keystream"),
    ("ctr_precompute", "fused_common.cuh", "ctr_precompute"),
    ("key_expansion", "fused_common.cuh", "expand_key_lane"),
    ("out_stream", "fused_common.cuh", "put16"),
    ("out_stream", "fused_common.cuh", "put"),
    ("out_stream", "fused_common.cuh", "finish"),
    ("payload_load", "fused_common.cuh", "load_raw6"),
    ("payload_load", "fused_common.cuh", "load_raw6_inb"),
    ("payload_load", "fused_common.cuh", "extract16"),
    ("esp_packet_other", "k_fused.cu", "esp_packet"),
    ("sa_line_load", "k_fused.cu", "load_pkt_pre"),
    ("prologue_scan_rows", "k_fused.cu", "pipe_scan_rows"),
    ("prologue_warps", "k_fused.cu", "pipe_prologue"),
    ("lpt", "k_fused.cu", "lpt_place"),
    ("seq_scan_poll", "k_fused.cu", "pipe_sequence"),
    ("scan_columns", "internal.cuh", "scan_all_columns"),
    ("scan_columns", "internal.cuh", "scan_sa_column"),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("--kernel", default="k_fused_ring_pipe")
    a = ap.parse_args()
    rows = list(csv.reader(open(a.csv)))
    hdr = next(r for r in rows if r and r[0] == "Address")
    hi = {k: i for i, k in enumerate(hdr)}
    data = [r for r in rows[rows.index(hdr) + 1:] if r and r[0].startswith("0x")]
    stall_cols = [k for k in hdr if k.startswith("stall_") or k.startswith("Warp Stall Sampling")]
    ins = sass_hist.disassemble(a.kernel)
    if len(ins) != len(data):
        print(f"warning: {len(ins)} SASS instructions here vs {len(data)} in the capture", file=sys.stderr)
    ranges = {}
    for name, f, fn in REGIONS:
        path = os.path.join(sass_hist.CSRC, f)
        r = sass_hist.func_ranges(path, [fn]).get(fn)
        if r:
            ranges.setdefault((name, f, fn), r)
    samp = collections.Counter()
    execd = collections.Counter()
    reasons = collections.defaultdict(collections.Counter)
    reason_cols = [k for k in hdr if k not in ("Address", "Source") and "Sampling" not in k and
                   k.startswith("stall") or k in ()]
    total = 0
    for k, row in enumerate(data):
        fr = ins[k][1] if k < len(ins) else []
        reg = "other"
        best = None
        for (name, f, fn), rg in ranges.items():
            for depth, (ff, ln) in enumerate(fr):
                if ff == f and rg[0] <= ln <= rg[1]:
                    if best is None or depth < best[0]:
                        best = (depth, name)
                    break
        if best:
            reg = best[1]
        s = int(float(row[hi["Warp Stall Sampling (All Samples)"]] or 0))
        samp[reg] += s
        total += s
        execd[reg] += int(float(row[hi["Instructions Executed"]] or 0))
        op = row[hi["Source"]].split()[0] if row[hi["Source"]].split() else "?"
        if op.startswith("@"):
            op = row[hi["Source"]].split()[1]
        reasons[reg][op.split(".")[0]] += s
    tot_e = sum(execd.values())
    print(f"{'region':22s} {'samples%':>9s} {'inst%':>7s}  top opcodes by samples")
    for reg, s in samp.most_common():
        top = ", ".join(f"{o} {100.0 * n / max(s, 1):.0f}%" for o, n in reasons[reg].most_common(5))
        print(f"{reg:22s} {100.0 * s / total:8.1f}% {100.0 * execd[reg] / tot_e:6.1f}%  {top}")


if __name__ == "__main__":
    main()
