#!/usr/bin/env python
"""Tiny launches of every backend and body for compute-sanitizer
(scripts/sanitize.sh runs this under memcheck, racecheck, synccheck and
initcheck).  Sizes are small so the instrumented runs finish in seconds;
each launch is checked against the oracle so a tool-induced schedule change
that broke the result would show as FAIL too.

    python scripts/sanitize_targets.py [group ...]   groups: runtime gemv stencil tbc halo spmv wave
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main(groups):
    import numpy as np
    import torch
    import oracle as O
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, synth
    dev = "cuda"
    ok = True

    def check(name, got, ref, exact=False):
        nonlocal ok
        got = np.asarray(got, dtype=np.float64)
        ref = np.asarray(ref, dtype=np.float64)
        if exact:
            good = np.array_equal(got, ref)
        else:
            m = ref != 0
            good = bool(np.all(got[~m] == 0)) and (not m.any() or np.max(np.abs(got[m] - ref[m]) / np.abs(ref[m])) <= 1e-4)
        ok &= good
        print(("ok   " if good else "FAIL ") + name, flush=True)

    if "wave" in groups:                     # CC_K_JACOBI5_WAVE: mailboxes, chunk claims, steals, cp.async rings
        u0 = synth.matrix(4, 300, 250)
        for b, kw in (("agent", dict(order="col")), ("agent", dict(order="row", active_agents=3)),
                      ("identity", {}), ("static", dict(order="col", num_clusters=7)), ("default", {})):
            for fuse in (3, 8):
                a_ = torch.from_numpy(u0).to(dev)
                got = ops.jacobi5_wave(a_, torch.zeros_like(a_), 2 * fuse + 1, fuse=fuse, backend=b, **kw)
                torch.cuda.synchronize()
                check(f"jacobi5_wave {b} {kw} fuse={fuse}", got.cpu().numpy(), O.jacobi5_f32(u0, 2 * fuse + 1),
                      exact=True)
    if "runtime" in groups:
        for b in ("agent", "identity", "static", "default", "redirect"):
            cen, _, _, _ = ops.census(13, 11, b, "row", num_clusters=148 if b == "static" else 0)
            torch.cuda.synchronize()
            check(f"census {b}", cen.cpu().numpy(), np.ones(13 * 11), exact=True)
        cen, _, _, _ = ops.census(13, 11, "agent", "tile", tile=(2, 3), active_agents=1)
        torch.cuda.synchronize()
        check("census agent tile throttled", cen.cpu().numpy(), np.ones(13 * 11), exact=True)
    if "gemv" in groups:
        m, n = 70, 600
        A = synth.matrix(3, m, n)
        p, r = synth.uniform(11, n), synth.uniform(12, m)
        q_ref, s_ref = O.bicg(A, p, r)
        for b in ("agent", "identity", "static", "default"):
            q, s = ops.bicg(torch.from_numpy(A).to(dev), torch.from_numpy(p).to(dev), torch.from_numpy(r).to(dev),
                            backend=b, order="col", num_clusters=148 if b == "static" else 0)
            torch.cuda.synchronize()
            check(f"bicg {b}", np.concatenate([q.cpu(), s.cpu()]), np.concatenate([q_ref, s_ref]))
        x = synth.uniform(10, n)
        tmp_ref, y_ref = O.atax(A, x)
        for b in ("agent", "identity", "static"):
            tmp, y = ops.atax_fused(torch.from_numpy(A).to(dev), torch.from_numpy(x).to(dev), backend=b,
                                    order="row", num_clusters=148 if b == "static" else 0)
            torch.cuda.synchronize()
            check(f"atax one-pass {b}", np.concatenate([tmp.cpu(), y.cpu()]), np.concatenate([tmp_ref, y_ref]))
    if "stencil" in groups:
        u0 = synth.matrix(4, 70, 100)
        for b in ("agent", "identity", "static", "default"):
            a = torch.from_numpy(u0).to(dev)
            out = ops.jacobi5(a, torch.zeros_like(a), 3, backend=b, order="row", num_clusters=148 if b == "static" else 0)
            torch.cuda.synchronize()
            check(f"jacobi {b}", out.cpu().numpy(), O.jacobi5_f32(u0, 3), exact=True)
        for K in (2, 3, 4):                      # fused sweeps (Jacobi5MultiBody<K>)
            for b in ("agent", "static"):
                a = torch.from_numpy(u0).to(dev)
                out = ops.jacobi5(a, torch.zeros_like(a), 2 * K, fuse=K, backend=b, order="row",
                                  num_clusters=148 if b == "static" else 0)
                torch.cuda.synchronize()
                check(f"jacobi fuse={K} {b}", out.cpu().numpy(), O.jacobi5_f32(u0, 2 * K), exact=True)
        for R in (1, 3):
            K = 2 * R + 1
            w = synth.uniform(6, K * K).reshape(K, K)
            ref = O.conv2d(u0, w)
            for b in ("agent", "static", "default"):
                o = ops.conv2d(torch.from_numpy(u0).to(dev), w, backend=b, order="row",
                               num_clusters=148 if b == "static" else 0)
                torch.cuda.synchronize()
                check(f"conv{K} {b}", o.cpu().numpy(), ref)
    if "tbc" in groups:
        u0 = synth.matrix(5, 150, 100)
        for R in (1, 3):
            K = 2 * R + 1
            w = synth.uniform(6, K * K).reshape(K, K)
            ref = O.conv2d(u0, w)
            for C in (1, 2, 4):
                o = ops.conv2d(torch.from_numpy(u0).to(dev), w, backend="tbcluster", cluster_size=C)
                torch.cuda.synchronize()
                check(f"conv{K} tbcluster C={C}", o.cpu().numpy(), ref)
    if "halo" in groups:
        from paper_conf_asplos_lis0l0c17_b200 import shard
        rows, cols, G, T = 100, 64, 2, 4
        u0 = synth.matrix(4, rows, cols)
        sl = []
        for g in range(G):
            lo, hi, llo, lhi = shard.slab_range(rows, G, g, 1)
            a = torch.from_numpy(np.ascontiguousarray(u0[llo:lhi])).to(dev)
            sl.append(dict(a=a, b=torch.zeros_like(a), lo=lo, hi=hi, llo=llo,
                           ll=torch.zeros(cc.ll_words(cols), dtype=torch.int64, device=dev)))
        for s in range(T):
            for g, x in enumerate(sl):
                src, dst = (x["a"], x["b"]) if s % 2 == 0 else (x["b"], x["a"])
                up = sl[g - 1]["ll"].data_ptr() if g > 0 else None
                dn = sl[g + 1]["ll"].data_ptr() if g < G - 1 else None
                ops.jacobi5_halo(src, dst, 1, s, x["ll"], up, dn, backend="agent", order="row", max_agents=1)
        torch.cuda.synchronize()
        got = np.concatenate([x["a"][x["lo"] - x["llo"]: x["hi"] - x["llo"]].cpu().numpy() for x in sl])
        check("jacobi fused LL halo, 2 virtual slabs", got, O.jacobi5_f32(u0, T), exact=True)
    if "spmv" in groups:
        rp, col = synth.rmat_csr(7, 9, 8)
        val, x = synth.uniform(8, len(col)), synth.uniform(9, len(rp) - 1)
        ref = O.spmv_csr(rp, col, val, x)
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)
        for hot in (0, 32):
            Am = ops.SpmvMatrix(t(rp.astype(np.int32)), t(col.astype(np.int32)), t(val), hot=hot)
            for b in ("agent", "default"):
                y = ops.spmv(Am, t(x), backend=b, order="row")
                torch.cuda.synchronize()
                check(f"spmv {b} hot={hot}", y.cpu().numpy(), ref)
            for b in ("agent", "static"):           # shared-memory hub tier (CC_K_SPMV_SHUB)
                y = ops.spmv(Am, t(x), backend=b, order="row", shub=True, num_clusters=148 if b == "static" else 0)
                torch.cuda.synchronize()
                check(f"spmv shub {b} hot={hot}", y.cpu().numpy(), ref)
        rp, col = synth.rmat_csr(7, 14, 4)         # both tiers: more hubs than the shared tier holds
        val, x = synth.uniform(8, len(col)), synth.uniform(9, len(rp) - 1)
        Am = ops.SpmvMatrix(t(rp.astype(np.int32)), t(col.astype(np.int32)), t(val), hot=cc.SPMV_SHUB_SLOTS + 7)
        y = ops.spmv(Am, t(x), backend="agent", order="row", shub=True)
        torch.cuda.synchronize()
        check("spmv shub two tiers", y.cpu().numpy(), O.spmv_csr(rp, col, val, x))
    print("ALL OK" if ok else "SOME FAILED", flush=True)
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main(sys.argv[1:] or ["runtime", "gemv", "stencil", "tbc", "halo", "spmv"]))
