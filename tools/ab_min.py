"""Best-of-passes summary of a tools/ab_variants.py run log: python tools/ab_min.py LOG"""
import collections
import re
import sys

d = collections.defaultdict(lambda: collections.defaultdict(list))
v = None
for line in open(sys.argv[1]):
    m = re.match(r"variant (\S+)", line)
    if m:
        v = m.group(1)
        continue
    m = re.match(r"\s+cfg (\d+): ([\d.]+)", line)
    if m:
        d[v][m.group(1)].append(float(m.group(2)))
for v in d:
    print(f"{v:22s}", "  ".join(f"cfg {k}: {min(x):7.1f}" for k, x in sorted(d[v].items())))
