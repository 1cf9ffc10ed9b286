#!/usr/bin/env python
"""Summarise gpurun_out/ncu_<tag>/*.csv (scripts/ncu_suite.sh) into
profiles/ncu_<tag>_summary.{json,md}: per kernel variant the L2 sectors
(all, and SM-originated = srcunit_tex, split by op), L1 hit rate, DRAM bytes,
duration, and the reduction / speedup relative to the default CTA order.

    python scripts/ncu_summarize.py r01
"""
import csv
import glob
import json
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SUM = ["lts__t_sectors.sum", "lts__t_sectors_srcunit_tex.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
       "lts__t_sectors_srcunit_tex_op_write.sum", "lts__t_sectors_srcunit_tex_op_red.sum",
       "lts__t_sectors_srcunit_tex_op_atom.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
       "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum"]
AVG = ["l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active"]


def num(s):
    s = s.replace(",", "").strip()
    try:
        return float(s)
    except ValueError:
        return None


def parse(path):
    rows = list(csv.reader(l for l in open(path) if l.startswith('"')))
    if not rows:
        return None
    hdr = rows[0]
    ix = {h: i for i, h in enumerate(hdr)}
    per = defaultdict(dict)
    units = {}
    for r in rows[1:]:
        if len(r) < len(hdr):
            continue
        kid = r[ix["ID"]]
        per[kid][r[ix["Metric Name"]]] = num(r[ix["Metric Value"]])
        units[r[ix["Metric Name"]]] = r[ix["Metric Unit"]]
        per[kid]["_kernel"] = r[ix["Kernel Name"]]
    if not per:
        return None
    out = {"launches": len(per), "kernels": sorted({v["_kernel"][:60] for v in per.values()})}
    for m in SUM:
        vals = [v.get(m) for v in per.values() if v.get(m) is not None]
        scale = 1.0
        if m.startswith("dram__bytes"):
            u = units.get(m, "byte")
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(u, 1)
        if m == "gpu__time_duration.sum":
            u = units.get(m, "nsecond")
            scale = {"nsecond": 1e-3, "usecond": 1, "msecond": 1e3, "ns": 1e-3, "us": 1, "ms": 1e3}.get(u, 1e-3)
        out[m if m != "gpu__time_duration.sum" else "duration_us"] = sum(vals) * scale if vals else None
    for m in AVG:
        vals = [v.get(m) for v in per.values() if v.get(m) is not None]
        out[m] = sum(vals) / len(vals) if vals else None
    return out


def main(tag):
    d = os.path.join(ROOT, "gpurun_out", f"ncu_{tag}")
    res = {}
    for p in sorted(glob.glob(os.path.join(d, "*.csv"))):
        name = os.path.basename(p)[:-4]
        if name.startswith("bench_launches"):
            continue
        r = parse(p)
        if r:
            res[name] = r
    groups = defaultdict(dict)
    for name, r in res.items():
        k, var = name.split("_", 1)
        groups[k][var] = r
    table = []
    for k, vs in groups.items():
        base = vs.get("default")
        for var, r in vs.items():
            row = {"kernel": k, "variant": var, "duration_us": r["duration_us"],
                   "l2_sectors": r["lts__t_sectors.sum"], "l2_sectors_sm": r["lts__t_sectors_srcunit_tex.sum"],
                   "l2_read": r["lts__t_sectors_srcunit_tex_op_read.sum"],
                   "l2_red_atom": (r["lts__t_sectors_srcunit_tex_op_red.sum"] or 0) + (r["lts__t_sectors_srcunit_tex_op_atom.sum"] or 0),
                   "l1_hit_pct": r["l1tex__t_sector_hit_rate.pct"],
                   "dram_bytes": (r["dram__bytes_read.sum"] or 0) + (r["dram__bytes_write.sum"] or 0),
                   "warps_active_pct": r["sm__warps_active.avg.pct_of_peak_sustained_active"]}
            if base and var != "default":
                bs = base["lts__t_sectors_srcunit_tex.sum"]
                row["l2_sm_sector_reduction_vs_default"] = 1 - r["lts__t_sectors_srcunit_tex.sum"] / bs if bs else None
                row["ncu_speedup_vs_default"] = base["duration_us"] / r["duration_us"] if r["duration_us"] else None
            table.append(row)
    dram = {f"{r['kernel']}_{r['variant']}": r["dram_bytes"] for r in table}
    out = {"tag": tag, "note": "ncu --metrics (cache-control all: L2 flushed before each replay), one launch "
           "per variant after one warm-up; atax = 2 launches summed.  l2_sectors_sm = lts__t_sectors_srcunit_tex "
           "(SM-originated; excludes L2<->L2 fabric traffic of the two dies).", "rows": table,
           "dram_bytes_per_launch": dram}
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    json.dump(out, open(os.path.join(ROOT, "profiles", f"ncu_{tag}_summary.json"), "w"), indent=1)
    lines = [f"# ncu summary {tag}", "", out["note"], "",
             "| kernel | variant | us | L2 sectors (SM) | reads | red+atom | L1 hit % | DRAM MB | warps act % | L2(SM) reduction | ncu speedup |",
             "|---|---|---|---|---|---|---|---|---|---|---|"]
    f = lambda x, p=1: "-" if x is None else (f"{x:.{p}f}" if isinstance(x, float) else str(x))
    for r in table:
        lines.append(f"| {r['kernel']} | {r['variant']} | {f(r['duration_us'])} | {f(r['l2_sectors_sm'], 0)} | "
                     f"{f(r['l2_read'], 0)} | {f(r['l2_red_atom'], 0)} | {f(r['l1_hit_pct'])} | {f(r['dram_bytes'] / 1e6)} | "
                     f"{f(r['warps_active_pct'])} | {f(r.get('l2_sm_sector_reduction_vs_default'), 3)} | "
                     f"{f(r.get('ncu_speedup_vs_default'), 3)} |")
    open(os.path.join(ROOT, "profiles", f"ncu_{tag}_summary.md"), "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r01")
