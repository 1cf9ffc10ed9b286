#!/usr/bin/env python
"""Print {metric: value} of each kernel in ncu --csv --metrics log files."""
import csv
import sys

for path in sys.argv[1:]:
    rows = list(csv.reader(open(path)))
    hdr = [r for r in rows if r and r[0] == "ID"]
    if not hdr:
        print(path, "(no data)")
        continue
    h = hdr[0]
    out = {}
    for r in rows:
        if len(r) == len(h) and r[0] != "ID":
            d = dict(zip(h, r))
            out.setdefault(d["Kernel Name"][:30], {})[d["Metric Name"]] = d["Metric Value"]
    for k, m in out.items():
        print(path.split("/")[-1], k, {n.split("__", 1)[1][:34]: v for n, v in m.items()})
