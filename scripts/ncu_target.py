#!/usr/bin/env python
"""Launch one kernel variant a few times for ncu (each launch is tagged with an
NVTX-free marker: the variant runs `--reps` launches after `--warm` warm-ups).

    python scripts/ncu_target.py --kernel bicg --backend agent --order col [--reps 2]
Kernels: matvec atax bicg mvt jacobi jwave conv3 conv7 spmv.  Sizes are the BASELINE
configs (jacobi: one sweep of 16384^2).
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kernel", required=True)
    ap.add_argument("--backend", default="agent")
    ap.add_argument("--order", default=None)
    ap.add_argument("--tile", default=None)
    ap.add_argument("--active", type=int, default=0)
    ap.add_argument("--stages", type=int, default=0)
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--staging", default="default")
    ap.add_argument("--cluster", type=int, default=2)
    ap.add_argument("--clusters", type=int, default=0, help="num_clusters M of the plan (static backend)")
    ap.add_argument("--l2", default=None, help="l2_hint name (ctaclust.L2_HINTS)")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--warm", type=int, default=1)
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--hot", type=int, default=0, help="spmv: hub-column form with this many hub slots")
    ap.add_argument("--fuse", type=int, default=1, help="jacobi: sweeps per launch (cc_jacobi5_args.fuse)")
    ap.add_argument("--persist-x", action="store_true", help="spmv: x L2-persisting (cc_l2_persist)")
    ap.add_argument("--small", action="store_true",
                    help="reduced problem (categorizer probe, P:2275): n/4 matrices, scale-18 SpMV")
    a = ap.parse_args()
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    kw = dict(backend=a.backend, active_agents=a.active, stages=a.stages, batch=a.batch, staging=a.staging)
    if a.order:
        kw["order"] = a.order
    if a.tile:
        kw["tile"] = tuple(int(t) for t in a.tile.split("x"))
    if a.backend == "tbcluster":
        kw["cluster_size"] = a.cluster
    if a.clusters:
        kw["num_clusters"] = a.clusters
    if a.l2:
        kw["l2_hint"] = a.l2
    dev = "cuda"
    k = a.kernel
    if k == "matvec":
        n = 1024
        A = synth.matrix(1, n, n, backend="torch", device=dev)
        x = synth.uniform(2, n, backend="torch", device=dev)
        y = torch.zeros(n, device=dev)
        fn = lambda: ops.matvec(A, x, y, **kw)
    elif k in ("atax", "bicg", "mvt", "atax_fused"):
        n = 4096 if a.small else 16384
        A = synth.matrix(3, n, n, backend="torch", device=dev)
        v = lambda s: synth.uniform(s, n, backend="torch", device=dev)
        x, p, r, y1, y2, x1, x2 = v(10), v(11), v(12), v(15), v(16), v(13), v(14)
        bufs = (torch.empty(n, device=dev), torch.empty(n, device=dev))
        fn = {"atax": lambda: ops.atax(A, x, out=bufs, **kw),
              "atax_fused": lambda: ops.atax_fused(A, x, out=bufs, **kw),
              "bicg": lambda: ops.bicg(A, p, r, out=bufs, **kw),
              "mvt": lambda: ops.mvt(A, y1, y2, x1, x2, **kw)}[k]
    elif k == "jacobi":
        N = 4096 if a.small else 16384
        a_ = synth.matrix(4, N, N, backend="torch", device=dev)
        b_ = torch.empty_like(a_)
        fn = lambda: ops.jacobi5(a_, b_, a.fuse, fuse=a.fuse, **kw)   # one launch of `fuse` sweeps
    elif k == "jwave":
        N = 4096 if a.small else 16384
        a_ = synth.matrix(4, N, N, backend="torch", device=dev)
        b_ = torch.empty_like(a_)
        kw.pop("stages"); kw.pop("staging")
        fn = lambda: ops.jacobi5_wave(a_, b_, a.fuse, fuse=a.fuse, **kw)   # one launch of `fuse` sweeps
    elif k in ("conv3", "conv7"):
        N, R = (2048 if a.small else 8192), (1 if k == "conv3" else 3)
        img = synth.matrix(5, N, N, backend="torch", device=dev)
        out = torch.empty_like(img)
        w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
        w = w / w.sum()
        fn = lambda: ops.conv2d(img, w, out=out, **kw)
    elif k == "spmv":
        rp, col = synth.rmat_csr(7, 18 if a.small else a.scale, 16, backend="torch", device=dev)
        val = synth.uniform(8, col.numel(), backend="torch", device=dev)
        x = synth.uniform(9, rp.numel() - 1, backend="torch", device=dev)
        Am = ops.SpmvMatrix(rp, col, val, hot=a.hot)
        y = torch.empty(rp.numel() - 1, device=dev)
        if a.persist_x:
            from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
            cc.l2_persist(x)
        if a.backend == "cusparse":          # vendor library, for context only
            Acsr = torch.sparse_csr_tensor(rp, col, val, (rp.numel() - 1, rp.numel() - 1))
            fn = lambda: torch.mv(Acsr, x)
        else:
            fn = lambda: ops.spmv(Am, x, y, **kw)
    elif k in ("hist", "hist_skewed"):
        n = 1 << (28 if a.small else 30)
        data = synth.bytes_u8(31, n, kind="skewed" if k == "hist_skewed" else "uniform", backend="torch", device=dev)
        counts = torch.empty(64, dtype=torch.int32, device=dev)
        fn = lambda: ops.hist64(data, counts, **kw)
    else:
        raise SystemExit(f"unknown kernel {k}")
    torch.cuda.synchronize()
    for _ in range(a.warm + a.reps):
        fn()
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
