#!/usr/bin/env python
"""Probe: TILE orders whose consecutive positions are vertical neighbours
(TILE(1,2), (1,4), (2,2)) vs ROW, default and identity on conv 3x3 / Jacobi
(one sweep), graph timing.  python scripts/vpair_probe.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench_suite as B  # noqa: E402


def main():
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    o = torch.empty_like(img)
    w = synth.uniform(6, 9).reshape(3, 3)
    w = w / w.sum()
    J = 16384
    a = synth.matrix(4, J, J, backend="torch", device="cuda")
    b = torch.empty_like(a)
    cases = {"conv3": (lambda kw: ops.conv2d(img, w, out=o, **kw), 8 * N * N),
             "jacobi": (lambda kw: ops.jacobi5(a, b, 1, **kw), 8 * J * J)}
    variants = [("default", dict(backend="default")), ("identity", dict(backend="identity")),
                ("row", dict(backend="agent", order="row"))]
    for t in ((1, 2), (1, 4), (2, 2), (2, 4), (4, 2), (8, 2)):
        variants.append((f"tile{t[0]}x{t[1]}", dict(backend="agent", order="tile", tile=t)))
    for name, (fn, nbytes) in cases.items():
        d = None
        print(f"== {name}")
        for vn, kw in variants:
            ms = B.graph_ms(lambda: fn(kw), 10, 10)
            d = d or ms
            print(f"   {vn:12s} {ms:.4f} ms  x{d / ms:.3f}  frac {nbytes / (ms * 1e-3) / 1e9 / B._peak():.3f}", flush=True)


if __name__ == "__main__":
    main()
