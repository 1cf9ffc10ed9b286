#!/usr/bin/env python
"""Summarise the bench launch list (scripts/ncu_bench.sh TAG) into
profiles/TAG/bench_launches_summary.md: launches, total / mean duration and
share of each of our kernels.

    python scripts/ncu_launches_summary.py r04
"""
import csv
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main(tag):
    src = os.path.join(ROOT, "gpurun_out", f"ncu_{tag}", "bench_launches.csv")
    rows = list(csv.reader(open(src)))
    h = [r for r in rows if r and r[0] == "ID"][0]
    tot, cnt = defaultdict(float), defaultdict(int)
    for r in rows:
        if len(r) == len(h) and r[0] != "ID":
            d = dict(zip(h, r))
            if d["Metric Name"] != "gpu__time_duration.sum":
                continue
            v = float(d["Metric Value"].replace(",", ""))
            v *= {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(d["Metric Unit"], 1e-3)
            tot[d["Kernel Name"]] += v
            cnt[d["Kernel Name"]] += 1
    all_us = sum(tot.values())
    out = [f"# bench.py launch list under ncu (our kernels only; gpu__time_duration.sum, --clock-control none, "
           f"cold-cache serialised: compare shares)", "",
           f"Command: `ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:k_(agent|default|redirect|static)' "
           f"python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-parity` (scripts/ncu_bench.sh {tag}). The timed "
           f"step is the agent (COL) ATAX+BICG+MVT; the default-order (TMA and direct) steps and the identity control "
           f"are timed after it in the same run.", "",
           "| kernel | launches | total us | mean us | share |", "|---|---|---|---|---|"]
    for k in sorted(tot, key=lambda k: -tot[k]):
        out.append(f"| `{k}` | {cnt[k]} | {tot[k]:.1f} | {tot[k] / cnt[k]:.1f} | {tot[k] / all_us:.3f} |")
    dst = os.path.join(ROOT, "profiles", tag, "bench_launches_summary.md")
    os.makedirs(os.path.dirname(dst), exist_ok=True)
    open(dst, "w").write("\n".join(out) + "\n")
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r04")
