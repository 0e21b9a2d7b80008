#!/usr/bin/env python
"""Top SASS instructions by warp-stall samples of an ncu report (--set full):

    python tools/ncu_hot_sass.py REPORT.ncu-rep"""
import csv, sys, subprocess
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[1]
i_addr, i_src, i_all = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
data = rows[2:]
tot = sum(int(r[i_all] or 0) for r in data if len(r) > i_all)
# find BAR / WARPSYNC / sleep instructions with most samples
top = sorted(data, key=lambda r: -int(r[i_all] or 0))[:25]
print("total samples", tot)
for r in top:
    print(r[i_addr][-5:], r[i_all], r[i_src].strip()[:70])
