#!/usr/bin/env python
"""Round-2 A/B experiments (one box, graph-timed like bench_suite):
  spmv   hub-column form (inspector slots 0 / 4K / 16K / 32K / 64K) x backends
  stencil TILE(2, h) orders (vertical runs of merged pairs) vs ROW / identity / default
    python scripts/exp_r10.py spmv|stencil out.json
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench_suite as B  # noqa: E402


def spmv():
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    rp, col = synth.rmat_csr(7, 24, 16, backend="torch", device="cuda")
    n, nnz = rp.numel() - 1, col.numel()
    val = synth.uniform(8, nnz, backend="torch", device="cuda")
    x = synth.uniform(9, n, backend="torch", device="cuda")
    y = torch.empty(n, device="cuda")
    nbytes = 8 * nnz + 4 * (n + 1) + 8 * n
    out = {}
    for hot in [int(h) for h in os.environ.get("EXP_SPMV_HOTS", "0,4096,16384,32768,65536").split(",")]:
        Am = ops.SpmvMatrix(rp, col, val, hot=hot)
        variants = [("default", dict(backend="default")), ("agent-row", dict(backend="agent", order="row")),
                    ("identity", dict(backend="identity")),
                    ("static-row-m5", dict(backend="static", order="row", num_clusters=5 * 148))]
        r = B.measure(variants, lambda kw: ops.spmv(Am, x, y, **kw), 20, nbytes, graph=True, inner=B.GRAPH_INNER)
        out[f"hot{hot}"] = r
        print(hot, [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
        del Am
        torch.cuda.empty_cache()
    return out


def spmv_persist():
    """SpMV with x (64 MiB) held L2-persisting through an access-policy window
    (cc_l2_persist) vs without; eager launches on one stream (the window is a
    stream attribute), 5 per event pair"""
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, synth
    rp, col = synth.rmat_csr(7, 24, 16, backend="torch", device="cuda")
    n, nnz = rp.numel() - 1, col.numel()
    val = synth.uniform(8, nnz, backend="torch", device="cuda")
    x = synth.uniform(9, n, backend="torch", device="cuda")
    y = torch.empty(n, device="cuda")
    nbytes = 8 * nnz + 4 * (n + 1) + 8 * n
    out = {}
    for hot in (0, 16384):
        Am = ops.SpmvMatrix(rp, col, val, hot=hot)
        variants = [("default", dict(backend="default")), ("agent-row", dict(backend="agent", order="row")),
                    ("identity", dict(backend="identity"))]
        for persist in (False, True):
            cc.l2_persist(x if persist else None, 1.0)
            r = B.measure(variants, lambda kw: ops.spmv(Am, x, y, **kw), 20, nbytes, inner=5)
            out[f"hot{hot}-persist{int(persist)}"] = r
            print(hot, persist, [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
        cc.l2_persist(None)
    return out


def spmv_control():
    """SpMV data-related class: (1) the no-locality control -- the same R-MAT
    graph with its vertices randomly relabelled; (2) an
    inspector-built USER order -- logical CTAs (merge-path blocks) sorted by
    the mean column they gather, so blocks reading similar x regions share a
    cluster (P:1771 'customized partition provided by users')."""
    import numpy as np
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    rp, col = synth.rmat_csr(7, 24, 16, backend="torch", device="cuda")
    n, nnz = rp.numel() - 1, col.numel()
    val = synth.uniform(8, nnz, backend="torch", device="cuda")
    x = synth.uniform(9, n, backend="torch", device="cuda")
    y = torch.empty(n, device="cuda")
    nbytes = 8 * nnz + 4 * (n + 1) + 8 * n
    out = {}
    Am = ops.SpmvMatrix(rp, col, val)
    # inspector USER order over the logical CTAs
    part = Am.part.cpu().numpy().astype(np.int64)
    rph = rp.cpu().numpy().astype(np.int64)
    colh = col.cpu().numpy().astype(np.int64)
    IPC = 4096
    nb = part.size - 1
    d0 = np.arange(nb, dtype=np.int64) * IPC
    y0 = d0 - part[:-1]                             # first nonzero of each block
    y1 = np.minimum(d0 + IPC, n + nnz) - part[1:]
    csum = np.concatenate([[0], np.cumsum(colh)])
    cnt = np.maximum(y1 - y0, 1)
    mean_col = (csum[np.minimum(y1, nnz)] - csum[np.minimum(y0, nnz)]) / cnt
    user = np.argsort(mean_col, kind="stable").astype(np.int32)
    variants = [("default", dict(backend="default")), ("agent-row", dict(backend="agent", order="row")),
                ("identity", dict(backend="identity")),
                ("agent-user-meancol", dict(backend="agent", order="user", user_order=user))]
    r = B.measure(variants, lambda kw: ops.spmv(Am, x, y, **kw), 20, nbytes, graph=True, inner=B.GRAPH_INNER)
    out["rmat"] = r
    print("rmat", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    del Am
    # no-locality control: relabel every vertex by a random permutation
    perm = torch.from_numpy(synth.random_permutation(3, n)).cuda()
    rows_of = torch.repeat_interleave(torch.arange(n, device="cuda"), (rp[1:] - rp[:-1]).long())
    keys = perm[rows_of] * n + perm[col.long()]
    keys, idx = torch.sort(keys)
    val2 = val[idx]
    del rows_of, idx
    r2 = (keys // n)
    col2 = (keys % n).to(torch.int32)
    del keys
    counts = torch.bincount(r2, minlength=n)
    rp2 = torch.zeros(n + 1, dtype=torch.int64, device="cuda")
    torch.cumsum(counts, 0, out=rp2[1:])
    Ap = ops.SpmvMatrix(rp2.to(torch.int32), col2, val2)
    variants = [("default", dict(backend="default")), ("agent-row", dict(backend="agent", order="row")),
                ("identity", dict(backend="identity"))]
    r = B.measure(variants, lambda kw: ops.spmv(Ap, x, y, **kw), 20, nbytes, graph=True, inner=B.GRAPH_INNER)
    out["rmat_permuted"] = r
    print("rmat_permuted", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    return out


def stencil():
    import numpy as np
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    out = {}
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    o = torch.empty_like(img)
    w = synth.uniform(6, 9).reshape(3, 3)
    w = (w / w.astype(np.float64).sum()).astype(np.float32)
    tiles = [(2, 2), (2, 4), (2, 8), (2, 16), (4, 4)]
    variants = [("default", dict(backend="default")), ("default-direct", dict(backend="default", staging="direct")),
                ("identity", dict(backend="identity")), ("agent-row", dict(backend="agent", order="row"))] + \
               [(f"agent-tile{tw}x{th}", dict(backend="agent", order="tile", tile=(tw, th))) for tw, th in tiles]
    r = B.measure(variants, lambda kw: ops.conv2d(img, w, out=o, **kw), 20, 8 * N * N, graph=True, inner=B.GRAPH_INNER)
    out["conv3"] = r
    print("conv3", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    del img, o
    M = 16384
    a = synth.matrix(4, M, M, backend="torch", device="cuda")
    b = a.clone()
    r = B.measure(variants, lambda kw: ops.jacobi5(a, b, 2, **kw), 10, 2 * 8 * M * M, graph=True, inner=5)
    out["jacobi"] = r
    print("jacobi", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    return out


def tbc():
    """thread-block-cluster (TMA multicast) backend vs default / identity / agent, conv 3x3 and 7x7"""
    import numpy as np
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    out = {}
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    o = torch.empty_like(img)
    for R in ((1,) if os.environ.get("EXP_CONV3_ONLY") else (1, 3)):
        K = 2 * R + 1
        w = synth.uniform(6, K * K).reshape(K, K)
        w = (w / w.astype(np.float64).sum()).astype(np.float32)
        variants = [("default", dict(backend="default")), ("identity", dict(backend="identity")),
                    ("agent-row", dict(backend="agent", order="row"))] + \
                   [(f"tbc{c}", dict(backend="tbcluster", cluster_size=c)) for c in (1, 2, 4, 8)]
        if R == 3:
            variants.append(("static-row-m7", dict(backend="static", order="row", num_clusters=7 * 148)))
        r = B.measure(variants, lambda kw: ops.conv2d(img, w, out=o, **kw), 20, 8 * N * N, graph=True,
                      inner=B.GRAPH_INNER)
        out[f"conv{K}"] = r
        print(f"conv{K}", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    return out


def panel():
    """ROW clusters over vertical panels: TILE(tw, gy) orders (panel-major, row-major inside a panel)"""
    import numpy as np
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    out = {}
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    o = torch.empty_like(img)
    w = synth.uniform(6, 9).reshape(3, 3)
    w = (w / w.astype(np.float64).sum()).astype(np.float32)
    v3 = [("default", dict(backend="default")), ("identity", dict(backend="identity")),
          ("agent-row", dict(backend="agent", order="row"))] + \
         [(f"agent-panel{tw}", dict(backend="agent", order="tile", tile=(tw, 256))) for tw in (32, 64, 128)]
    r = B.measure(v3, lambda kw: ops.conv2d(img, w, out=o, **kw), 20, 8 * N * N, graph=True, inner=B.GRAPH_INNER)
    out["conv3"] = r
    print("conv3", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    del img, o
    M = 16384
    a = synth.matrix(4, M, M, backend="torch", device="cuda")
    b = a.clone()
    vj = [("default", dict(backend="default")), ("identity", dict(backend="identity")),
          ("agent-row", dict(backend="agent", order="row"))] + \
         [(f"agent-panel{tw}", dict(backend="agent", order="tile", tile=(tw, 512))) for tw in (32, 64, 128, 256)]
    r = B.measure(vj, lambda kw: ops.jacobi5(a, b, 2, **kw), 10, 2 * 8 * M * M, graph=True, inner=5)
    out["jacobi"] = r
    print("jacobi", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    return out


def conv7():
    """conv 7x7 variants of the agent / static backends (tile-shape A/B builds)"""
    import numpy as np
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    o = torch.empty_like(img)
    w = synth.uniform(6, 49).reshape(7, 7)
    w = (w / w.astype(np.float64).sum()).astype(np.float32)
    variants = [("default", dict(backend="default")), ("identity", dict(backend="identity")),
                ("agent-row", dict(backend="agent", order="row"))] + \
               [(f"static-row-m{m}", dict(backend="static", order="row", num_clusters=m * 148))
                for m in [int(v) for v in os.environ.get("EXP_C7_M", "3,4,6,7,8").split(",")]]
    r = B.measure(variants, lambda kw: ops.conv2d(img, w, out=o, **kw), 20, 8 * N * N, graph=True, inner=B.GRAPH_INNER)
    fl = 2 * 49 * (N - 6) ** 2
    for v in r["rows"]:
        v["tflops"] = round(fl / (v["ms"] * 1e-3) / 1e12, 2)
    print("conv7", [(v["variant"], v["ms"], v["tflops"]) for v in r["rows"]], flush=True)
    return {"conv7": r}


def hist():
    """HST (S8(f)3): default vs persistent variants, uniform and skewed bytes,
    1 GiB (round 2 measured per-lane privatised 16-bit counters here: 0.53-0.74
    ms against 0.29 ms for the shared-atomic default -- rejected and removed,
    profiles/r11/exp/hist_privatised.json)"""
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    out = {}
    n = 1 << 30
    for kind in ("uniform", "skewed"):
        data = synth.bytes_u8(31, n, kind=kind, backend="torch", device="cuda")
        counts = torch.empty(64, dtype=torch.int32, device="cuda")
        variants = [("default", dict(backend="default")), ("agent-row", dict(backend="agent", order="row")),
                    ("agent-row-s2", dict(backend="agent", order="row", stages=2)),
                    ("identity", dict(backend="identity")),
                    ("static-row-m1", dict(backend="static", order="row", num_clusters=148))]
        r = B.measure(variants, lambda kw: ops.hist64(data, counts, **kw), 20, n, graph=True, inner=B.GRAPH_INNER)
        out[kind] = r
        print(kind, [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
        del data
    return out


def _stripe_order(gx, gy, sw):
    """USER order of column stripes sw tiles wide: v runs stripe by stripe,
    row-major inside a stripe -- with one cluster per stripe every SM walks
    down its own columns while all of them stay on the same band of rows"""
    import numpy as np
    s, by, k = np.meshgrid(np.arange(gx // sw), np.arange(gy), np.arange(sw), indexing="ij")
    return (by * gx + s * sw + k).reshape(-1).astype(np.int32)


def stripe():
    """column-striped clusters (one stripe per SM, lock-step row band) vs
    identity / ROW / default: conv 3x3 8192^2 (128 stripes of 2 tiles) and
    Jacobi 16384^2 (128 stripes of 4 tiles)"""
    import numpy as np
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    out = {}
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    o = torch.empty_like(img)
    w = synth.uniform(6, 9).reshape(3, 3)
    w = (w / w.astype(np.float64).sum()).astype(np.float32)
    u3 = _stripe_order(256, 256, 2)
    base = [("default", dict(backend="default")), ("identity", dict(backend="identity")),
            ("agent-row", dict(backend="agent", order="row"))]
    v3 = base + [("agent-stripe", dict(backend="agent", order="user", user_order=u3, num_clusters=128))] + \
        [(f"static-stripe-s{st}", dict(backend="static", order="user", user_order=u3, num_clusters=128, stages=st))
         for st in (4, 8, 12)]
    r = B.measure(v3, lambda kw: ops.conv2d(img, w, out=o, **kw), 20, 8 * N * N, graph=True, inner=B.GRAPH_INNER)
    out["conv3"] = r
    print("conv3", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    del img, o
    M = 16384
    a = synth.matrix(4, M, M, backend="torch", device="cuda")
    b = a.clone()
    uj = _stripe_order(512, 512, 4)
    vj = base + [("agent-stripe", dict(backend="agent", order="user", user_order=uj, num_clusters=128))] + \
        [(f"static-stripe-s{st}", dict(backend="static", order="user", user_order=uj, num_clusters=128, stages=st))
         for st in (4, 8, 12)]
    r = B.measure(vj, lambda kw: ops.jacobi5(a, b, 2, **kw), 10, 2 * 8 * M * M, graph=True, inner=5)
    out["jacobi"] = r
    print("jacobi", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    return out


def spmv_shub():
    """hub array in each agent's shared memory (CC_K_SPMV_SHUB) vs the L1 hub
    form and plain CSR; EXP_SHUB_HOTS lists the hub sizes (<= the build's
    capacity)"""
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    rp, col = synth.rmat_csr(7, 24, 16, backend="torch", device="cuda")
    n, nnz = rp.numel() - 1, col.numel()
    val = synth.uniform(8, nnz, backend="torch", device="cuda")
    x = synth.uniform(9, n, backend="torch", device="cuda")
    y = torch.empty(n, device="cuda")
    nbytes = 8 * nnz + 4 * (n + 1) + 8 * n
    out = {}
    A0 = ops.SpmvMatrix(rp, col, val, hot=16384)
    base = [("default-l1hub16k", dict(backend="default")), ("agent-row-l1hub16k", dict(backend="agent", order="row")),
            ("identity-l1hub16k", dict(backend="identity"))]
    r = B.measure(base, lambda kw: ops.spmv(A0, x, y, **kw), 20, nbytes, graph=True, inner=B.GRAPH_INNER)
    out["l1hub16k"] = r
    print("l1hub16k", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
    del A0
    for hot in [int(h) for h in os.environ.get("EXP_SHUB_HOTS", "16384,32768,43008").split(",")]:
        Am = ops.SpmvMatrix(rp, col, val, hot=hot)
        variants = [("default-l1hub", dict(backend="default")),
                    ("shub-agent-row", dict(backend="agent", order="row", shub=True)),
                    ("shub-identity", dict(backend="identity", shub=True)),
                    ("shub-static-row-m1", dict(backend="static", order="row", num_clusters=148, shub=True)),
                    ("shub-agent-row-s12", dict(backend="agent", order="row", shub=True, stages=6, batch=4))]
        r = B.measure(variants, lambda kw: ops.spmv(Am, x, y, **kw), 20, nbytes, graph=True, inner=B.GRAPH_INNER)
        out[f"shub{hot}"] = r
        print(f"shub{hot}", [(v["variant"], v["ms"], v["frac_hbm"]) for v in r["rows"]], flush=True)
        del Am
        torch.cuda.empty_cache()
    return out


if __name__ == "__main__":
    what, path = sys.argv[1], sys.argv[2]
    res = {"spmv": spmv, "stencil": stencil, "tbc": tbc, "panel": panel, "conv7": conv7,
           "spmv_control": spmv_control, "hist": hist, "spmv_persist": spmv_persist,
           "stripe": stripe, "spmv_shub": spmv_shub}[what]()
    json.dump(res, open(path, "w"), indent=1)
