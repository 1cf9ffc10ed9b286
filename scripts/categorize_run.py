#!/usr/bin/env python
"""Run the section 4.4 / Fig. 11 categorizer on every kernel (GPU box).

Probe: ncu metrics (categorize.NCU_METRICS) of default / RD-X / RD-Y and, for
the stencils, L1-on (cp.async.ca staging) / L1-off (TMA staging), at a reduced
problem size ("better to reduce the problem size").  Then the verdict
and its optimisation set, tuned in-process at the BASELINE size.

    python scripts/categorize_run.py gpurun_out/categorize.json [--only k1,k2]
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

KERNELS = {  # name: (ncu_target kernel, launches per call, has L1/TMA staging, writes shifted reads)
    "matvec": ("matvec", 1, False, False), "atax": ("atax", 2, False, False), "bicg": ("bicg", 1, False, False),
    "mvt": ("mvt", 1, False, False), "jacobi5": ("jacobi", 1, True, False), "conv3x3": ("conv3", 1, True, False),
    "conv7x7": ("conv7", 1, True, False), "spmv": ("spmv", 1, False, False),
    "hist64": ("hist", 1, False, False)}


def ncu_probe(out_dir, name, kern, per, args):
    from paper_conf_asplos_lis0l0c17_b200 import categorize as C
    csvf = os.path.join(out_dir, f"{name}.csv")
    cmd = ["ncu", "--metrics", ",".join(C.NCU_METRICS), "--clock-control", "none", "-k",
           "regex:k_(agent|default|redirect)", "-s", str(per), "-c", str(per), "--csv", "--log-file", csvf,
           sys.executable, os.path.join(ROOT, "scripts", "ncu_target.py"), "--small", "--warm", "1", "--reps", "1",
           "--kernel", kern] + args
    subprocess.run(cmd, stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL, timeout=600, check=False)
    return C.probe_from_ncu_csv(csvf)


def full_size_runner(name):
    import numpy as np
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ops, synth
    if name == "matvec":
        n = 1024
        A = synth.matrix(1, n, n, backend="torch", device="cuda")
        x = synth.uniform(2, n, backend="torch", device="cuda")
        y = torch.zeros(n, device="cuda")
        return (lambda **kw: ops.matvec(A, x, y, **kw)), 50
    if name in ("atax", "bicg", "mvt"):
        n = 16384
        A = synth.matrix(3, n, n, backend="torch", device="cuda")
        v = lambda s: synth.uniform(s, n, backend="torch", device="cuda")
        x, p, r, y1, y2, x1, x2 = v(10), v(11), v(12), v(15), v(16), v(13), v(14)
        bufs = (torch.empty(n, device="cuda"), torch.empty(n, device="cuda"))
        return {"atax": lambda **kw: ops.atax(A, x, out=bufs, **kw),
                "bicg": lambda **kw: ops.bicg(A, p, r, out=bufs, **kw),
                "mvt": lambda **kw: ops.mvt(A, y1, y2, x1, x2, **kw)}[name], 1
    if name == "jacobi5":
        N = 16384
        a = synth.matrix(4, N, N, backend="torch", device="cuda")
        b = torch.empty_like(a)
        return (lambda **kw: ops.jacobi5(a, b, 10, **kw)), 1
    if name.startswith("conv"):
        R = 1 if name == "conv3x3" else 3
        N = 8192
        img = synth.matrix(5, N, N, backend="torch", device="cuda")
        out = torch.empty_like(img)
        w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
        w = (w / w.sum()).astype(np.float32)
        return (lambda **kw: ops.conv2d(img, w, out=out, **kw)), 1
    if name == "spmv":
        rp, col = synth.rmat_csr(7, 24, 16, backend="torch", device="cuda")
        val = synth.uniform(8, col.numel(), backend="torch", device="cuda")
        x = synth.uniform(9, rp.numel() - 1, backend="torch", device="cuda")
        Am = ops.SpmvMatrix(rp, col, val)
        y = torch.empty(rp.numel() - 1, device="cuda")
        return (lambda **kw: ops.spmv(Am, x, y, **kw)), 1
    if name == "hist64":
        data = synth.bytes_u8(31, 1 << 30, backend="torch", device="cuda")
        counts = torch.empty(64, dtype=torch.int32, device="cuda")
        return (lambda **kw: ops.hist64(data, counts, **kw)), 1
    raise KeyError(name)


def graph_ms(fn, reps, inner):
    """Per-launch time of `inner` launches captured in one CUDA graph (microsecond
    kernels: keeps the host launch rate out of the measurement)."""
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import categorize as C
    fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(inner):
            fn()
    return C.time_ms(g.replay, reps) / inner


def main():
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import categorize as C, ctaclust as cc
    out = sys.argv[1]
    only = None
    if "--only" in sys.argv:
        only = sys.argv[sys.argv.index("--only") + 1].split(",")
    probe_dir = os.path.join(os.path.dirname(out) or ".", "categorize_ncu")
    os.makedirs(probe_dir, exist_ok=True)
    res = {}
    for name, (kern, per, l1, wsr) in KERNELS.items():
        if only and name not in only:
            continue
        pr = lambda tag, args: ncu_probe(probe_dir, f"{name}_{tag}", kern, per, args)
        sig = C.Signals(default=pr("default", ["--backend", "default"]),
                        rd_x=pr("rd-x", ["--backend", "redirect", "--order", "col"]),
                        rd_y=pr("rd-y", ["--backend", "redirect", "--order", "row"]),
                        l1_on=pr("l1-on", ["--backend", "default", "--staging", "l1"]) if l1 else None,
                        l1_off=pr("l1-off", ["--backend", "default", "--staging", "tma"]) if l1 else None,
                        writes_shifted_reads=wsr)
        v = C.categorize(sig)
        run, inner = full_size_runner(name)
        timer = (lambda fn, reps: graph_ms(fn, reps, inner)) if inner > 1 else (lambda fn, reps: C.time_ms(fn, reps))
        kname = {"jacobi5": "jacobi5", "conv3x3": "conv2d", "conv7x7": "conv2d"}.get(name, name)
        tr = C.tune(run, C.candidates(v, cc.max_agents(kname), has_staging=l1), reps=5, timer=timer)
        res[name] = {"signals": {k: (vars(p) if p is not None else None) for k, p in vars(sig).items()
                                 if k != "writes_shifted_reads"},
                     "verdict": v.as_dict(), "best": tr.best, "best_kw": tr.best_kw,
                     "best_ms": round(tr.best_ms, 5), "default_ms": round(tr.default_ms, 5),
                     "speedup_vs_default": round(tr.speedup, 4),
                     "table": [(n, round(ms, 5)) for n, ms in tr.table]}
        print(name, v.category, v.partition, tr.best, f"x{tr.speedup:.3f}", flush=True)
        del run
        torch.cuda.empty_cache()
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
