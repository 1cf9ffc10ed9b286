#!/usr/bin/env python
"""Per-kernel registers / spills / smem from an nvcc -Xptxas -v log.
    python scripts/ptxas_regs.py build_ptxas.log [old_log]   (diff when two)"""
import re
import subprocess
import sys


def parse(text):
    out, cur = {}, None
    for line in text.splitlines():
        m = re.search(r"Compiling entry function '([^']+)'", line)
        if m:
            cur = m.group(1)
            continue
        m = re.search(r"(\d+) bytes spill stores", line)
        if m and cur:
            out.setdefault(cur, {})["spill"] = int(m.group(1))
        m = re.search(r"Used (\d+) registers", line)
        if m and cur:
            out.setdefault(cur, {})["regs"] = int(m.group(1))
    return out


def demangle(names):
    try:
        r = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True)
        return dict(zip(names, r.stdout.splitlines()))
    except Exception:
        return {n: n for n in names}


if __name__ == "__main__":
    new = parse(open(sys.argv[1]).read())
    old = parse(open(sys.argv[2]).read()) if len(sys.argv) > 2 else None
    dm = demangle(list(new))
    for k, v in sorted(new.items(), key=lambda kv: dm[kv[0]]):
        o = old.get(k) if old else None
        tag = "" if not o else ("" if o == v else f"   (was {o.get('regs')} regs, {o.get('spill')} spill)")
        if old is None or tag:
            print(f"{v.get('regs'):4} regs {v.get('spill'):4} spill  {dm[k][:110]}{tag}")
