#!/usr/bin/env python
"""Summarise tools/gpu_ab.sh output: median ms per (config, alg, lib), skipping the first (warm-up) query."""
import re
import statistics
import sys

cur, rows = None, {}
for line in open(sys.argv[1]):
    m = re.match(r"== (\S+) (\S+) \S*/(\S+)\.so", line)
    if m:
        cur = m.groups()
        rows[cur] = []
        continue
    m = re.search(r"ms=([\d.]+)", line)
    if m and cur:
        rows[cur].append(float(m.group(1)))
for (cfg, alg, lib), v in rows.items():
    w = v[1:] if len(v) > 1 else v
    print(f"{cfg:4s} {alg:5s} {lib:14s} median {statistics.median(w) if w else float('nan'):8.3f} ms  all {v}")
