#!/usr/bin/env python
"""Agent ROW knob sweep for the stencils (batch, ring depth, active agents,
L2 hint) against default order and the identity control, same box, graph
timing.  python scripts/stencil_sweep.py out.json"""
import itertools
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench_suite as B  # noqa: E402


def main(out):
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    res = {}
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    o = torch.empty_like(img)
    w = synth.uniform(6, 9).reshape(3, 3)
    w = w / w.sum()
    J = 16384
    a = synth.matrix(4, J, J, backend="torch", device="cuda")
    b = torch.empty_like(a)
    cases = {"conv3": (lambda kw: ops.conv2d(img, w, out=o, **kw), 8 * N * N, 10),
             "jacobi": (lambda kw: ops.jacobi5(a, b, 1, **kw), 8 * J * J, 10)}
    variants = [("default", dict(backend="default")), ("identity", dict(backend="identity"))]
    for bt, st, act, hint in itertools.product((1, 2, 4, 8), (2, 4, 6), (0, 3), ("none", "reuse_last")):
        variants.append((f"row-b{bt}-s{st}-a{act}-{hint}",
                         dict(backend="agent", order="row", batch=bt, stages=st, active_agents=act, l2_hint=hint)))
    for name, (fn, nbytes, inner) in cases.items():
        rows = []
        for vn, kw in variants:
            try:
                ms = B.graph_ms(lambda: fn(kw), 10, inner)
                rows.append((vn, ms))
            except Exception as e:  # noqa: BLE001
                rows.append((vn, None))
                print(vn, "error", repr(e)[:120])
        res[name] = rows
        d = dict(rows)["default"]
        print(f"== {name}")
        for vn, ms in sorted(rows, key=lambda r: r[1] or 1e9)[:12]:
            print(f"   {vn:34s} {ms:.4f} ms  x{d / ms:.3f}  frac {nbytes / (ms * 1e-3) / 1e9 / B._peak():.3f}")
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1])
