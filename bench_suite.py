#!/usr/bin/env python
"""bench_suite.py -- every BASELINE config, clustered vs default CTA order.

For each reuse kernel this times the default hardware order ("BSL") --
both with the library's TMA-staged body and with the plain direct-load body,
the faster of the two being the comparator -- against the agent runtime with
the config's clustering ("CLU"), throttled agents ("CLU+TOT"), staging
variants (TMA = L1-bypassing "BPS", L1-allocating cp.async, direct loads), ring
depth, the persistence-only control (identity order) and redirection ("RD").
Reports ms, algorithmic GB/s (fraction of the measured HBM copy peak) and the
speedup over the best default.  L2-sector reductions come from the ncu
captures (scripts/ncu_suite.sh -> profiles/).

    python bench_suite.py out.json [--only matvec,atax,jacobi,conv,spmv] [--quick]
"""
from __future__ import annotations

import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)


def _peak():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    except Exception:
        return 6650.0


def time_ms(fn, reps, warm=3, inner=1):
    import torch
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(inner):
            fn()
        b.record()
        b.synchronize()
        out.append(a.elapsed_time(b) / inner)
    out.sort()
    return out[len(out) // 2]


def graph_ms(fn, reps, inner):
    """Time `inner` launches captured in one CUDA graph (removes the Python /
    host launch overhead that dominates microsecond kernels)."""
    import torch
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(inner):
            fn()
    g.replay()
    torch.cuda.synchronize()
    return time_ms(g.replay, reps, warm=1) / inner


# Sub-millisecond kernels are timed as GRAPH_INNER back-to-back launches
# replayed from one CUDA graph: with one eagerly launched call per event pair
# the host-side marshalling of the call (ctypes arguments, plan lookup,
# cc_launch validation) sits inside the timed interval.
GRAPH_INNER = 10
VARIANT_FILTER = None   # --variants REGEX: keep matching rows (plus the default-order rows)


def measure(variants, fn, reps, nbytes, extra=None, warm=3, inner=1, graph=False, context=None):
    """`context`: {name: callable} vendor-library timings of the same
    computation (cuBLAS / cuDNN / cuSPARSE via torch), reported as lib-* rows
    for absolute context; they are not part of the default/clustered
    comparison."""
    rows = []
    if VARIANT_FILTER:
        import re
        variants = [(n, kw) for n, kw in variants if n.startswith("default") or re.search(VARIANT_FILTER, n)]
        context = None
    for name, kw in variants:
        ms = graph_ms(lambda: fn(kw), reps, inner) if graph else time_ms(lambda: fn(kw), reps, warm=warm, inner=inner)
        gbs = nbytes / (ms * 1e-3) / 1e9
        d = {"variant": name, "ms": round(ms, 5), "GBps": round(gbs, 1), "frac_hbm": round(gbs / _peak(), 4)}
        if extra:
            d.update(extra(ms))
        rows.append(d)
    for name, cfn in (context or {}).items():
        try:
            ms = graph_ms(cfn, reps, inner) if graph else time_ms(cfn, reps, warm=warm, inner=inner)
            gbs = nbytes / (ms * 1e-3) / 1e9
            rows.append({"variant": "lib-" + name, "ms": round(ms, 5), "GBps": round(gbs, 1),
                         "frac_hbm": round(gbs / _peak(), 4)})
        except Exception as e:  # context only
            rows.append({"variant": "lib-" + name, "error": repr(e)[:200]})
    best_def = min(r["ms"] for r in rows if r["variant"].startswith("default"))
    for r in rows:
        if "ms" not in r:
            continue
        r["speedup_vs_best_default"] = round(best_def / r["ms"], 4)
    return {"bytes": nbytes, "best_default_ms": best_def, "rows": rows}


def variants_for(order, tile=(1, 1), stencil=False):
    o = dict(order=order, tile=tile) if order == "tile" else dict(order=order)
    tag = f"{order}{tile[0]}x{tile[1]}" if order == "tile" else order
    v = [("default", dict(backend="default")),
         ("default-direct", dict(backend="default", staging="direct")),
         (f"agent-{tag}", dict(backend="agent", **o)),
         (f"agent-{tag}-direct", dict(backend="agent", staging="direct", **o)),
         (f"agent-{tag}-tot1", dict(backend="agent", active_agents=1, **o)),
         (f"agent-{tag}-tot2", dict(backend="agent", active_agents=2, **o)),
         (f"agent-{tag}-s2", dict(backend="agent", stages=2, **o)),
         ("identity", dict(backend="identity")),
         ("identity-direct", dict(backend="identity", staging="direct")),
         (f"redirect-{tag}", dict(backend="redirect", **o))]
    if stencil:
        v += [("default-l1", dict(backend="default", staging="l1")),
              (f"agent-{tag}-l1", dict(backend="agent", staging="l1", **o)),
              ("agent-row", dict(backend="agent", order="row")),
              ("agent-col", dict(backend="agent", order="col")),
              ("agent-tile4x4", dict(backend="agent", order="tile", tile=(4, 4))),
              ("agent-row-l1", dict(backend="agent", order="row", staging="l1")),
              (f"agent-{tag}-s6", dict(backend="agent", stages=6, **o))]
    return v


def f2_variants(order, tile=(1, 1), l1_staging=None):
    """S§8(f)2: L2 eviction-priority hints on the clustered agent (CLU+BPS) and a
    carveout sweep on the variant that relies on L1 (`l1_staging`)."""
    o = dict(order=order, tile=tile) if order == "tile" else dict(order=order)
    tag = f"{order}{tile[0]}x{tile[1]}" if order == "tile" else order
    v = [(f"agent-{tag}-l2first", dict(backend="agent", l2_hint="stream_first", **o)),
         (f"agent-{tag}-l2last", dict(backend="agent", l2_hint="reuse_last", **o)),
         (f"agent-{tag}-l2both", dict(backend="agent", l2_hint="both", **o))]
    if l1_staging:
        for cv in (0, 25, 50, 100):
            v.append((f"agent-{tag}-{l1_staging}-cv{cv}", dict(backend="agent", staging=l1_staging, carveout=cv, **o)))
    return v


def halo_hint_variants():
    """Stencils: CC_L2_HINT_HALO_LAST (the rows the next tile row re-reads as its
    top halo evict_last, the rest evict_first), alone and with the output
    stores evict_first."""
    return [("agent-row-l2halo", dict(backend="agent", order="row", l2_hint="halo_last")),
            ("agent-row-l2halo-sf", dict(backend="agent", order="row", l2_hint="halo_last_stream_first")),
            ("agent-tile8x8-l2halo", dict(backend="agent", order="tile", tile=(8, 8), l2_hint="halo_last"))]


def static_variants(kernel, order, tile=(1, 1), ks=None):
    """CC_BACKEND_AGENT_STATIC rows: M = SMs x k clusters, CTA i runs cluster i
    (binding by construction: no %smid, queue atomics or stealing)."""
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    nsm = cc.device_info(0)["num_sms"]
    amax = cc.max_agents(kernel)
    o = dict(order=order, tile=tile) if order == "tile" else dict(order=order)
    tag = f"{order}{tile[0]}x{tile[1]}" if order == "tile" else order
    ks = sorted(set(ks or (1, 2, amax)))
    return [(f"static-{tag}-m{k}", dict(backend="static", num_clusters=nsm * k, **o)) for k in ks if k <= 4 * amax]


def band_variants(gy):
    """Stencil orders that keep a global front (like the identity control) while
    clustering.  rowfront: the static backend with one cluster per tile row (M =
    gy): every row is a CTA walking left to right, all rows at once, so a tile's
    vertical neighbours are processed at the same moment by the CTAs of the
    rows above and below (halo re-reads hit L2).  band: TILE blocks one or a
    few tile columns wide and the grid tall, each SM walking its band top to
    bottom."""
    return [("static-rowfront-M" + str(gy), dict(backend="static", order="row", num_clusters=gy)),
            ("static-rowfront-M" + str(2 * gy), dict(backend="static", order="row", num_clusters=2 * gy)),
            ("static-rowfront-M" + str(gy // 2), dict(backend="static", order="row", num_clusters=gy // 2)),
            ("agent-band4-m128", dict(backend="agent", order="tile", tile=(4, gy), num_clusters=128)),
            ("static-band1-m512", dict(backend="static", order="tile", tile=(1, gy), num_clusters=512)),
            ("static-band2-m256", dict(backend="static", order="tile", tile=(2, gy), num_clusters=256)),
            ("agent-tile16x16", dict(backend="agent", order="tile", tile=(16, 16))),
            ("agent-tile32x8", dict(backend="agent", order="tile", tile=(32, 8)))]


def interleaved_order(gx, gy, M, c):
    """USER order for a time-aligned row clustering: the row-major sequence is
    cut into chunks of c horizontally adjacent tiles and chunk k goes to
    cluster k mod M, so every cluster holds co-located pairs (merged staging)
    while all clusters sweep the image top to bottom together (the vertical
    halo is re-read from L2 while it is still there)."""
    import numpy as np
    V = gx * gy
    K = (V + c - 1) // c
    seq = []
    for i in range(M):
        for k in range(i, K, M):
            seq.extend(range(k * c, min(V, (k + 1) * c)))
    out = np.asarray(seq, dtype=np.int32)
    assert out.size == V
    return out


def ilv_variants(gx, gy, cs=(2, 4, 8), static_ks=(2, 4)):
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    nsm = cc.device_info(0)["num_sms"]
    v = [(f"agent-ilv-c{c}", dict(backend="agent", user_order=interleaved_order(gx, gy, nsm, c))) for c in cs]
    v += [(f"static-ilv-c2-m{k}", dict(backend="static", num_clusters=nsm * k,
                                        user_order=interleaved_order(gx, gy, nsm * k, 2))) for k in static_ks]
    return v


def suite_matvec(quick):
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    n = 1024
    A = synth.matrix(1, n, n, backend="torch", device="cuda")
    x = synth.uniform(2, n, backend="torch", device="cuda")
    y = torch.zeros(n, device="cuda")
    v = variants_for("row") + [("agent-col", dict(backend="agent", order="col")),
                               ("agent-row-m1s4b4", dict(backend="agent", order="row", max_agents=1, stages=4, batch=4)),
                               ("agent-row-m2s3b2", dict(backend="agent", order="row", max_agents=2, stages=3, batch=2))] \
        + static_variants("matvec", "row", ks=(1, 2, 3, 4, 7)) \
        + [("static-row-m1-s6", dict(backend="static", order="row", num_clusters=148, stages=6)),
           ("static-row-m2-s4", dict(backend="static", order="row", num_clusters=296, stages=4))]
    r = measure(v, lambda kw: ops.matvec(A, x, y, **kw), 20 if quick else 50, 4 * n * n + 8 * n, inner=50, graph=True,
                context={"cublas-mv": lambda: torch.mv(A, x, out=y)})
    r["config"] = "tiled fp32 matvec n=1024, 32x32 tiles (32x32 grid), L2-resident; 50 launches per CUDA graph"
    return r


def suite_atax(quick):
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    n = 16384
    A = synth.matrix(3, n, n, backend="torch", device="cuda")
    v = lambda s: synth.uniform(s, n, backend="torch", device="cuda")
    x, p, r, y1, y2, x1, x2 = v(10), v(11), v(12), v(15), v(16), v(13), v(14)
    tmp, y, q, s = (torch.empty(n, device="cuda") for _ in range(4))
    Ab = 4 * n * n
    kernels = {
        "atax": (lambda kw: ops.atax(A, x, out=(tmp, y), **kw), 2 * Ab + 16 * n),
        "bicg": (lambda kw: ops.bicg(A, p, r, out=(q, s), **kw), Ab + 16 * n),
        "mvt": (lambda kw: ops.mvt(A, y1, y2, x1, x2, **kw), Ab + 24 * n),
    }
    variants = variants_for("col") + [("agent-row", dict(backend="agent", order="row")),
                                      ("agent-col-s3", dict(backend="agent", order="col", stages=3))] \
        + f2_variants("col", l1_staging="direct") + static_variants("bicg", "col") + static_variants("bicg", "row", ks=(3,))
    ctx = {"atax": {"cublas-2xmv": lambda: torch.mv(A.t(), torch.mv(A, x, out=tmp), out=y)},
           "bicg": {"cublas-2xmv": lambda: (torch.mv(A, p, out=q), torch.mv(A.t(), r, out=s))},
           "mvt": {"cublas-2xmv": lambda: (x1.add_(torch.mv(A, y1)), x2.add_(torch.mv(A.t(), y2)))}}
    out = {k: measure(variants, fn, 5 if quick else 15, nb, context=ctx[k], graph=True, inner=GRAPH_INNER) for k, (fn, nb) in kernels.items()}
    return {"config": "PolyBench ATAX/BICG/MVT fp32 n=16384, 32x256 tiles (64x512 grid)", "kernels": out}


def suite_jacobi(quick):
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    N, T = 16384, (20 if quick else 100)
    a = synth.matrix(4, N, N, backend="torch", device="cuda")
    b = torch.empty_like(a)
    v = variants_for("tile", (8, 8), stencil=True) + f2_variants("row") + f2_variants("tile", (8, 8), l1_staging="l1") \
        + static_variants("jacobi5", "row") + static_variants("jacobi5", "tile", (8, 8), ks=(4,)) + band_variants(N // 32) \
        + ilv_variants(N // 32, N // 32) + halo_hint_variants()
    r = measure(v, lambda kw: ops.jacobi5(a, b, T, **kw), 3, 8 * N * N * T,
                extra=lambda ms: {"ms_per_sweep": round(ms / T, 5)}, warm=1)
    r["config"] = f"2D 5-point Jacobi fp32 {N}x{N}, {T} sweeps, 32x32 tiles (512x512 grid)"
    return r


def suite_conv(quick):
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    out = torch.empty_like(img)
    res = {}
    for R in (1, 3):
        w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
        w = w / w.sum()
        flops = 2 * (2 * R + 1) ** 2 * (N - 2 * R) ** 2
        v = variants_for("tile", (8, 8), stencil=True) + [
            ("tbcluster-2", dict(backend="tbcluster", cluster_size=2)),
            ("tbcluster-4", dict(backend="tbcluster", cluster_size=4)),
            ("tbcluster-8", dict(backend="tbcluster", cluster_size=8))] \
            + f2_variants("row") + f2_variants("tile", (8, 8), l1_staging="l1") \
            + static_variants("conv2d", "row") + static_variants("conv2d", "tile", (8, 8), ks=(4,)) + band_variants(N // 32) \
            + ilv_variants(N // 32, N // 32) + halo_hint_variants()
        wt = torch.from_numpy(w).cuda().view(1, 1, 2 * R + 1, 2 * R + 1)
        img4 = img.view(1, 1, N, N)
        res[f"{2 * R + 1}x{2 * R + 1}"] = measure(
            v, lambda kw: ops.conv2d(img, w, out=out, **kw), 5 if quick else 20, 8 * N * N, graph=True, inner=GRAPH_INNER,
            extra=lambda ms: {"TFLOPs": round(flops / (ms * 1e-3) / 1e12, 2)},
            context={"cudnn-conv2d": lambda: torch.nn.functional.conv2d(img4, wt)})
        res[f"{2 * R + 1}x{2 * R + 1}"]["flops"] = flops
    return {"config": f"2D conv fp32 {N}x{N}, 32x32 tiles (256x256 grid)", "filters": res}


def suite_spmv(quick):
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    scale = 20 if quick else 24
    t0 = time.time()
    rp, col = synth.rmat_csr(7, scale, 16, backend="torch", device="cuda")
    gen_s = time.time() - t0
    rows_n = rp.numel() - 1
    nnz = col.numel()
    val = synth.uniform(8, nnz, backend="torch", device="cuda")
    x = synth.uniform(9, rows_n, backend="torch", device="cuda")
    Am = ops.SpmvMatrix(rp, col, val)
    y = torch.empty(rows_n, device="cuda")
    variants = [("default", dict(backend="default")), ("agent-row", dict(backend="agent", order="row")),
                ("agent-row-tot1", dict(backend="agent", order="row", active_agents=1)),
                ("agent-row-tot2", dict(backend="agent", order="row", active_agents=2)),
                ("agent-row-tot4", dict(backend="agent", order="row", active_agents=4)),
                ("agent-row-b8", dict(backend="agent", order="row", batch=8)),
                ("agent-row-s1", dict(backend="agent", order="row", stages=1)),
                ("agent-row-s4", dict(backend="agent", order="row", stages=4)),
                ("identity", dict(backend="identity")), ("identity-s1", dict(backend="identity", stages=1)),
                ("redirect-row", dict(backend="redirect", order="row"))] + f2_variants("row") \
        + [(f"{b}-cv{cv}", dict(backend=b, carveout=cv, **({"order": "row"} if b == "agent" else {})))
           for b in ("default", "agent") for cv in (0, 25, 50, 100)] + static_variants("spmv", "row")
    Acsr = torch.sparse_csr_tensor(rp, col, val, (rows_n, rows_n))
    r = measure(variants, lambda kw: ops.spmv(Am, x, y, **kw), 5 if quick else 20,
                8 * nnz + 4 * (rows_n + 1) + 8 * rows_n, graph=True, inner=GRAPH_INNER,
                context={"cusparse-spmv": lambda: torch.mv(Acsr, x)})
    r["config"] = f"CSR SpMV fp32 R-MAT scale {scale} ef 16: {rows_n} rows, {nnz} nnz (gen {gen_s:.1f}s)"
    return r


def suite_hist(quick):
    """S8(f)3: the paper's HST (64-bin histogram, data-related) -- CTA
    prefetching with the agent's ordered stream (PFH) vs default order."""
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    n = 1 << (28 if quick else 30)
    counts = torch.empty(64, dtype=torch.int32, device="cuda")
    res = {}
    for kind in ("uniform", "skewed"):
        data = synth.bytes_u8(31, n, kind=kind, backend="torch", device="cuda")
        v = [("default", dict(backend="default")), ("default-direct", dict(backend="default", staging="direct")),
             ("agent-row", dict(backend="agent", order="row")),
             ("agent-row-s1", dict(backend="agent", order="row", stages=1)),
             ("agent-row-s2", dict(backend="agent", order="row", stages=2)),
             ("agent-row-s4", dict(backend="agent", order="row", stages=4)),
             ("agent-row-direct", dict(backend="agent", order="row", staging="direct")),
             ("agent-row-tot1", dict(backend="agent", order="row", active_agents=1)),
             ("agent-col", dict(backend="agent", order="col")),
             ("identity", dict(backend="identity")), ("redirect-row", dict(backend="redirect", order="row"))] \
            + static_variants("hist64", "row")
        res[kind] = measure(v, lambda kw: ops.hist64(data, counts, **kw), 5 if quick else 20, n + 256, graph=True,
                            inner=GRAPH_INNER)
        del data
    return {"config": f"64-bin histogram (HST, R24) of {n} bytes, 32 KiB per logical CTA", "inputs": res}


def suite_slabs(quick):
    """Config 3's slab sharding (S§8(e)) on one GPU: G = 8 virtual slabs of the
    16384^2 Jacobi, 100 sweeps, each slab's sweep a separate launch, the slabs'
    sweeps interleaved on one stream (captured in one CUDA graph).  Halo
    exchange either fused into the sweep kernel (S§8(f)4, CC_K_JACOBI5_HALO:
    tagged peer stores into the neighbours' LL buffers) or done as separate device-to-device row copies after
    every sweep (the single-GPU stand-in for NCCL send/recv).  The unsharded
    sweep is the reference; the difference is the cost of sharding + exchange."""
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, shard, synth
    N, T, G = 16384, (20 if quick else 100), 8
    u = synth.matrix(4, N, N, backend="torch", device="cuda")
    slabs = []
    for g in range(G):
        lo, hi, llo, lhi = shard.slab_range(N, G, g, 1)
        a = u[llo:lhi].clone()
        slabs.append(dict(a=a, b=torch.empty_like(a), lo=lo, hi=hi, llo=llo, lhi=lhi,
                          ll=torch.zeros(cc.ll_words(N), dtype=torch.int64, device="cuda")))
    full_b = torch.empty_like(u)

    def fused(kw):
        for x in slabs:
            x["ll"].zero_()
        nb = lambda h: slabs[h]["ll"].data_ptr() if 0 <= h < G else None
        for s in range(T):
            for g, x in enumerate(slabs):
                src, dst = (x["a"], x["b"]) if s % 2 == 0 else (x["b"], x["a"])
                ops.jacobi5_halo(src, dst, 1, s, x["ll"], nb(g - 1), nb(g + 1), None, **kw)

    def copies(kw):
        for s in range(T):
            outs = []
            for x in slabs:
                src, dst = (x["a"], x["b"]) if s % 2 == 0 else (x["b"], x["a"])
                ops.jacobi5(src, dst, 1, **kw)
                outs.append(dst)
            for g in range(G - 1):                 # halo rows <- neighbours' owned boundary rows
                outs[g][-1].copy_(outs[g + 1][1])
                outs[g + 1][0].copy_(outs[g][-2])

    def nohalo(kw):                                # the sharded sweeps with no exchange at all (timing only)
        for s in range(T):
            for x in slabs:
                src, dst = (x["a"], x["b"]) if s % 2 == 0 else (x["b"], x["a"])
                ops.jacobi5(src, dst, 1, **kw)

    rows = []
    nbytes = 8 * N * N * T
    peak = _peak()
    for name, fn, kw in [("unsharded-agent-row", lambda kw: ops.jacobi5(u, full_b, T, **kw), dict(backend="agent", order="row")),
                         ("unsharded-identity", lambda kw: ops.jacobi5(u, full_b, T, **kw), dict(backend="identity")),
                         ("unsharded-default", lambda kw: ops.jacobi5(u, full_b, T, **kw), dict(backend="default")),
                         ("slabs8-fused-agent-row", fused, dict(backend="agent", order="row")),
                         ("slabs8-fused-identity", fused, dict(backend="identity")),
                         ("slabs8-fused-default", fused, dict(backend="default")),
                         ("slabs8-copies-agent-row", copies, dict(backend="agent", order="row")),
                         ("slabs8-copies-identity", copies, dict(backend="identity")),
                         ("slabs8-copies-default", copies, dict(backend="default")),
                         ("slabs8-noexchange-agent-row", nohalo, dict(backend="agent", order="row")),
                         ("slabs8-noexchange-identity", nohalo, dict(backend="identity"))]:
        ms = graph_ms(lambda: fn(kw), 3, 1)
        gbs = nbytes / (ms * 1e-3) / 1e9
        rows.append({"variant": name, "ms": round(ms, 4), "ms_per_sweep": round(ms / T, 5), "GBps": round(gbs, 1),
                     "frac_hbm": round(gbs / peak, 4)})
    best = min(r["ms"] for r in rows if r["variant"].startswith("unsharded"))
    for r in rows:
        r["speedup_vs_best_default"] = round(best / r["ms"], 4)       # here: vs the best unsharded run
    return {"config": f"Jacobi {N}^2 x {T} sweeps as {G} virtual slabs on one GPU (fused peer halo vs "
                      f"separate row copies; vs unsharded)", "bytes": nbytes, "rows": rows}


SUITES = {"matvec": suite_matvec, "atax": suite_atax, "jacobi": suite_jacobi, "conv": suite_conv, "spmv": suite_spmv, "hist": suite_hist,
          "slabs": suite_slabs}


def run(path, only=None, quick=False):
    import torch
    res = {"device": torch.cuda.get_device_name(0), "hbm_peak_GBps": _peak()}
    for k, fn in SUITES.items():
        if only and k not in only:
            continue
        t0 = time.time()
        try:
            res[k] = fn(quick)
        except Exception as e:  # keep the other configs
            res[k] = {"error": repr(e)}
        res[k]["wall_s"] = round(time.time() - t0, 1)
        torch.cuda.empty_cache()
        json.dump(res, open(path, "w"), indent=1)
    return res


def table(path):
    d = json.load(open(path))
    lines = []
    for k, v in d.items():
        if not isinstance(v, dict):
            continue
        groups = {k: v} if "rows" in v else {f"{k}/{kk}": vv for sub in ("kernels", "filters", "inputs") for kk, vv in v.get(sub, {}).items()}
        for g, vv in groups.items():
            lines.append(f"== {g}  {v.get('config', '')}")
            for r in vv.get("rows", []):
                if "ms" not in r:
                    lines.append(f"   {r['variant']:26s} {r.get('error', '')}")
                    continue
                sp = r.get("speedup_vs_best_default")
                lines.append(f"   {r['variant']:26s} {r['ms']:10.4f} ms {r['GBps']:8.1f} GB/s  frac {r['frac_hbm']:.3f}  x{sp:.3f}")
    return "\n".join(lines)


if __name__ == "__main__":
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("out")
    ap.add_argument("--only", default=None)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--variants", default=None, help="regex: time only matching variants (and default order)")
    a = ap.parse_args()
    VARIANT_FILTER = a.variants
    run(a.out, a.only.split(",") if a.only else None, a.quick)
    print(table(a.out))
