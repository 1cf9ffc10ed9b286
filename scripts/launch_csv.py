"""Per-kernel duration statistics from an ncu --csv launch list.
    python scripts/launch_csv.py file.csv [filter-substring]"""
import collections
import csv
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr]
    ki, vi, mi = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Name")
    d = collections.defaultdict(list)
    for r in rows[hdr + 1:]:
        if len(r) > vi and r[mi] == "gpu__time_duration.sum":
            d[r[ki]].append(float(r[vi].replace(",", "")) / 1000.0)
    return d


if __name__ == "__main__":
    d = load(sys.argv[1])
    flt = sys.argv[2] if len(sys.argv) > 2 else ""
    for k, v in d.items():
        if flt in k:
            print(f"{k[:70]:70s} n={len(v):4d} mean={sum(v) / len(v):8.2f} us  first8={sum(v[:8]) / min(8, len(v)):8.2f}"
                  f"  rest={sum(v[8:]) / max(1, len(v) - 8):8.2f}")
