#!/usr/bin/env python
"""bench.py -- locality-aware CTA clustering on B200, one BASELINE config per run.

Default (the headline, BASELINE config 2): PolyBench ATAX + BICG + MVT, fp32,
n = 16384, column clustering (the paper's X-partition for ATX/MVT/BC, Table 2
P:2297-2301) with the agent runtime, row-sharded over N GPUs.  `--config`
selects another BASELINE config through the same drivers (drivers.py):
jacobi (config 3, slab-sharded, boundary-first overlapped halo exchange),
conv3 / conv7 (config 4), spmv (config 5).

A step = one pass of the config's hot path over its whole input (ATAX: 4
streaming passes over the 1 GiB matrix; Jacobi: 100 sweeps).  `value` is
whole-job algorithmic HBM bytes per second; the same step in the default
hardware CTA order and in the persistence-only identity order is timed back
to back (`speedup_vs_default`, `speedup_vs_identity`).

    python bench.py [--config atax|jacobi|conv3|conv7|spmv] [--gpus N --steps K --warmup W]
                    [--impl reference] [--suite out.json]

Rules kept: W >= 3 warm-ups; K timed steps bracketed by barrier + synchronize,
CUDA events on the launching stream, max over ranks; every config's inputs
exceed L2 (126 MB) except where stated in `config.l2`; SM clocks and
throttle reasons sampled through NVML during the timed region.  The oracle
(oracle/, CPU) runs only in the cpu_baseline leg, the sampled parity probe
after the timed region (rank 0) and --impl reference.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "speedup & L2 sector reduction vs default CTA order; HBM GB/s vs roofline"
NSM = 148

# headline launch options per config (the measured best clustered variant,
# DESIGN.md §10), overridable from the command line
HEADLINE = {
    "atax": dict(backend="agent", order="col"),
    "jacobi": dict(backend="agent", order="col"),      # wave kernel (R34); the tile-fused one: ROW
    "conv3": dict(backend="agent", order="row"),
    "conv7": dict(backend="static", order="row", num_clusters=7 * NSM),
    "spmv": dict(backend="agent", order="row"),
}
WORKLOAD = {
    "atax": "ATAX+BICG+MVT fp32 n=16384 (BASELINE config 2)",
    "jacobi": "Jacobi 5-point fp32 16384x16384, 100 sweeps per step (BASELINE config 3)",
    "conv3": "conv2d 3x3 fp32 8192x8192 (BASELINE config 4)",
    "conv7": "conv2d 7x7 fp32 8192x8192 (BASELINE config 4)",
    "spmv": "CSR SpMV fp32 R-MAT scale 24, edge factor 16 (BASELINE config 5)",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="atax", choices=sorted(HEADLINE))
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=0, help="timed steps (default per config)")
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--size", "--n", dest="n", type=int, default=0,
                    help="problem size override (atax n, jacobi/conv side, spmv scale)")
    ap.add_argument("--iters", type=int, default=100, help="jacobi sweeps per step")
    ap.add_argument("--backend", default=None)
    ap.add_argument("--order", default=None)
    ap.add_argument("--active-agents", type=int, default=0)
    ap.add_argument("--stages", type=int, default=0)
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--staging", default="default", choices=["default", "tma", "direct", "l1"])
    ap.add_argument("--no-overlap", action="store_true", help="jacobi: exchange after the whole sweep")
    ap.add_argument("--fuse", type=int, default=0,
                    help="jacobi: sweeps per launch (0: 8 for the wave kernel, 3 for the tile-fused one)")
    ap.add_argument("--tile-rows", type=int, default=0,
                    help="jacobi wave: logical CTA height in rows (0 = 64; DESIGN §10.0)")
    ap.add_argument("--jkernel", choices=("wave", "tile"), default="wave",
                    help="jacobi: strip wavefronts carried across tiles (CC_K_JACOBI5_WAVE, R34) or tile-fused "
                         "sweeps (CC_K_JACOBI5, R32)")
    ap.add_argument("--halo", default="exchange", choices=["exchange", "fused"],
                    help="jacobi N > 1: NCCL halo exchange per sweep, or the fused peer-memory LL halo")
    ap.add_argument("--no-graph", action="store_true", help="eager launches instead of one CUDA graph per step")
    ap.add_argument("--hot", type=int, default=16384, help="spmv: hub slots of the inspector (0: plain CSR)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-parity", action="store_true")
    ap.add_argument("--no-ncu", action="store_true", help="skip the live ncu L2-sector / DRAM count of the step")
    ap.add_argument("--suite", default=None, help="also run every BASELINE config's variants, write JSON here")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "torch"],
                    help="N > 1 exchanges: the library's NCCL communicator (default) or torch.distributed/gloo "
                         "(tests only)")
    ap.add_argument("--same-device", action="store_true",
                    help="tests only: run every rank on GPU 0 (exercises the N > 1 code on a 1-GPU box)")
    a = ap.parse_args()
    if not a.steps:
        a.steps = {"atax": 100, "jacobi": 10, "conv3": 200, "conv7": 200, "spmv": 50}[a.config]
    return a


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return None


def jacobi_fuse(a):
    f = getattr(a, "fuse", 0) or 0
    return f if f > 0 else (8 if getattr(a, "jkernel", "tile") == "wave" else 3)


def sizes(a):
    if a.config == "atax":
        return {"n": a.n or 16384}
    if a.config == "jacobi":
        return {"side": a.n or 16384, "iters": a.iters}
    if a.config in ("conv3", "conv7"):
        return {"side": a.n or 8192, "R": 1 if a.config == "conv3" else 3}
    return {"scale": a.n or 24}


# ------------------------------------------------------------------ clocks
class Clocks:
    """SM clock and throttle reasons sampled through NVML every ~2 ms on a
    background thread while the timed region runs (nvidia-smi fallback)."""
    REASONS = {"hw_slowdown": 0x8, "hw_thermal_slowdown": 0x40, "sw_thermal_slowdown": 0x20,
               "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, torch_device):
        self.samples, self.reasons, self.err = [], 0, None
        self._stop = threading.Event()
        self.max_mhz = None
        try:
            import pynvml as N
            import torch
            N.nvmlInit()
            pr = torch.cuda.get_device_properties(torch_device)
            bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
            self.h = N.nvmlDeviceGetHandleByPciBusId(bus)
            self.N = N
            self.max_mhz = N.nvmlDeviceGetMaxClockInfo(self.h, N.NVML_CLOCK_SM)
        except Exception as e:
            self.h, self.err = None, repr(e)[:120]
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()

    def _run(self):
        while not self._stop.is_set() and self.h is not None:
            try:
                self.samples.append(self.N.nvmlDeviceGetClockInfo(self.h, self.N.NVML_CLOCK_SM))
                self.reasons |= int(self.N.nvmlDeviceGetCurrentClocksEventReasons(self.h))
            except Exception as e:
                self.err = repr(e)[:120]
                return
            time.sleep(0.002)

    def stop(self):
        self._stop.set()
        self.t.join(timeout=2)
        if self.h is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "samples": 0, "reasons": [f"nvml unavailable: {self.err}"]}
        s = sorted(self.samples)
        return {"sm_mhz": s[len(s) // 2] if s else None, "sm_max_mhz": self.max_mhz, "samples": len(s),
                "reasons": sorted(k for k, b in self.REASONS.items() if self.reasons & b), "source": "nvml"}


# ------------------------------------------------------------------ oracle legs (CPU)
def cpu_info():
    model = None
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return {"cpu_count": os.cpu_count(), "model": model}


def oracle_sample(cfg, sz, min_secs, omp=False):
    """The oracle (plain C, fp64) on a bounded sample of the config's workload,
    repeated until `min_secs` have passed.  Returns (GB/s in the config's
    algorithmic bytes, secs, description, threads)."""
    import numpy as np
    import oracle as O
    from paper_conf_asplos_lis0l0c17_b200 import drivers, synth
    O.use_openmp(omp)
    t0 = time.perf_counter()
    done, nbytes = 0, 0
    if cfg == "atax":
        n, rows = sz["n"], 4096
        A = synth.matrix(3, rows, n)
        x, p = synth.uniform(10, n), synth.uniform(11, n)
        r, x1 = synth.uniform(12, rows), synth.uniform(13, rows)
        x2, y1, y2 = synth.uniform(14, n), synth.uniform(15, n), synth.uniform(16, rows)
        t0 = time.perf_counter()
        while done < 1 or time.perf_counter() - t0 < min_secs:
            O.atax(A, x)
            O.bicg(A, p, r)
            O.mvt(A, x1, x2, y1, y2)
            done += 1
        nbytes = done * drivers.atax_family_bytes(rows, n)["total"]
        desc = f"ATAX+BICG+MVT on rows 0..{rows - 1} of the {n}x{n} matrix x{done}"
    elif cfg == "jacobi":
        rows, cols = 1024, sz["side"]
        u0 = synth.matrix(4, rows, cols)
        t0 = time.perf_counter()
        while done < 1 or time.perf_counter() - t0 < min_secs:
            O.jacobi5(u0, 4)
            done += 4
        nbytes = done * 8 * rows * cols
        desc = f"{done} fp64 sweeps of a {rows}x{cols} slab"
    elif cfg in ("conv3", "conv7"):
        R = sz["R"]
        rows, cols = 1024, sz["side"]
        img = synth.matrix(5, rows, cols)
        w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
        t0 = time.perf_counter()
        while done < 1 or time.perf_counter() - t0 < min_secs:
            O.conv2d(img, w)
            done += 1
        nbytes = done * 8 * rows * cols
        desc = f"{done} x {2 * R + 1}x{2 * R + 1} conv of a {rows}x{cols} block"
    else:
        scale = min(sz["scale"], 20)
        rp, col = synth.rmat_csr(7, scale, 16)
        val, xv = synth.uniform(8, len(col)), synth.uniform(9, len(rp) - 1)
        t0 = time.perf_counter()
        while done < 1 or time.perf_counter() - t0 < min_secs:
            O.spmv_csr(rp, col, val, xv)
            done += 1
        nbytes = done * (8 * len(col) + 4 * len(rp) + 8 * (len(rp) - 1))
        desc = f"{done} x SpMV of R-MAT scale {scale} ({len(col)} nnz)"
    dt = time.perf_counter() - t0
    thr = O.omp_threads()
    O.use_openmp(False)
    return nbytes / dt / 1e9, dt, desc, thr


def run_reference(a):
    """--impl reference: the oracle as it stands, all host cores (OpenMP
    build), on a bounded sample of the config per step; rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if int(os.environ.get("WORLD_SIZE", "1")) > 1 and rank != 0:
        return 0
    sz = sizes(a)
    steps = max(1, min(a.steps, 10))
    oracle_sample(a.config, sz, 0.0, omp=True)                 # warm-up (builds, page-in)
    tot_b, tot_t, desc, thr = 0.0, 0.0, "", 1
    for _ in range(steps):
        gbs, dt, desc, thr = oracle_sample(a.config, sz, 1.0, omp=True)
        tot_b += gbs * dt
        tot_t += dt
    gbs = tot_b / tot_t
    ci = cpu_info()
    line = {"impl": "reference", "metric": METRIC, "value": round(gbs, 4), "unit": "GB/s", "n_gpus": a.gpus,
            "steps": steps, "warmup": a.warmup, "ms_per_step": round(1e3 * tot_t / steps, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (counter-hash generators, same seeds as the GPU arm)",
            "config": {"workload": WORKLOAD[a.config], "sample": desc + " per step (oracle, fp64, OpenMP)"},
            "cpu_baseline": {"value": round(gbs, 4), "unit": "GB/s", "cores": thr, "kind": "oracle",
                             "sample": desc, "cpu": ci},
            "e2e": {"value": round(gbs, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def parity_probe(cfg, D, world):
    """Sampled comparison of this rank's results with the oracle (after the
    timed region, on a fresh step from the initial state)."""
    import numpy as np
    import oracle as O
    from paper_conf_asplos_lis0l0c17_b200 import synth

    def rel(got, ref):
        got = np.asarray(got, dtype=np.float64)
        ref = np.asarray(ref, dtype=np.float64)
        m = ref != 0
        return float(np.max(np.abs(got[m] - ref[m]) / np.abs(ref[m]))) if m.any() else 0.0

    if cfg == "atax":
        n, lo, hi = D.n, D.lo, D.hi
        rows = [lo, lo + 1, (lo + hi) // 2, hi - 1]
        cols = [0, 1, n // 3, n - 1]
        errs = {}
        Ar = np.stack([synth.uniform(3, n, i * n) for i in rows])
        xv, p, y1 = synth.uniform(10, n), synth.uniform(11, n), synth.uniform(15, n)
        x1_0 = synth.uniform_at(13, rows)
        errs["tmp"] = rel(D.tmp.cpu().numpy()[[i - lo for i in rows]], O.matvec(Ar, xv))
        errs["q"] = rel(D.q.cpu().numpy()[[i - lo for i in rows]], O.matvec(Ar, p))
        errs["x1"] = rel(D.x1.cpu().numpy()[[i - lo for i in rows]], x1_0 + O.matvec(Ar, y1))
        m = D.m_total
        Ac = np.stack([synth.uniform_at(3, np.arange(m) * n + j) for j in cols])   # columns as rows
        r, y2, x2_0 = synth.uniform(12, m), synth.uniform(16, m), synth.uniform_at(14, cols)
        errs["s"] = rel(D.s.cpu().numpy()[cols], O.matvec(Ac, r))
        errs["x2"] = rel(D.x2.cpu().numpy()[cols], x2_0 + O.matvec(Ac, y2))
        tmp_all = getattr(D, "tmp_all", None)
        if tmp_all is not None:                    # y = A^T tmp with the GPU's fp32 tmp (pass 2 alone)
            errs["y"] = rel(D.y.cpu().numpy()[cols], O.matvec(Ac, tmp_all.cpu().numpy()))
        return {"max_rel_err": max(errs.values()), "per_output": errs, "tol": 1e-4,
                "ok": bool(max(errs.values()) <= 1e-4), "sample": f"rows {rows}, cols {cols}"}
    if cfg == "jacobi":
        T, cols = D.iters, D.cols
        got = D.result().cpu().numpy()
        pts = [(D.lo, 5), (D.lo + 1, cols // 2), ((D.lo + D.hi) // 2, cols - 2), (D.hi - 1, 1), (D.hi - 1, cols // 3)]
        bad = 0
        for (r, c) in pts:                          # light cone of radius T around (r, c)
            r0, r1 = max(r - T, 0), min(r + T + 1, D.rows)
            c0, c1 = max(c - T, 0), min(c + T + 1, cols)
            win = np.stack([synth.uniform(4, c1 - c0, i * cols + c0) for i in range(r0, r1)])
            ref = O.jacobi5_f32(win, T)[r - r0, c - c0]
            bad += int(got[r - D.lo, c] != ref)
        return {"mismatches": bad, "points": len(pts), "ok": bad == 0, "criterion": "bit-exact vs fp32 oracle",
                "sample": "light cones of radius iters around 5 owned points"}
    if cfg in ("conv3", "conv7"):
        R, cols = D.R, D.cols
        got = D.result().cpu().numpy()
        errs = []
        rlo, rhi = max(D.lo, R), min(D.hi, D.rows - R) - 8       # 8-row blocks inside the owned rows
        for (r, c) in [(rlo, R), ((rlo + rhi) // 2, cols // 2), (rhi, cols - 1 - R - 16)]:
            r = min(max(r, rlo), rhi)
            img = np.stack([synth.uniform(5, 16 + 2 * R, i * cols + c - R) for i in range(r - R, r + 8 + R)])
            ref = O.conv2d(img, D.w)[R:R + 8, R:R + 16]
            errs.append(rel(got[r - D.lo: r - D.lo + 8, c: c + 16], ref))
        return {"max_rel_err": float(max(errs)), "ok": bool(max(errs) <= 1e-4), "tol": 1e-4,
                "sample": "3 blocks of 8x16 outputs"}
    if cfg == "spmv":
        rp = D.A.row_ptr.cpu().numpy()
        rows = sorted({0, 1, D.A.rows // 2, D.A.rows - 1} | {int(i) for i in np.argsort(np.diff(rp))[-3:]})
        col, val = D.A.col.cpu().numpy(), D.A.val.cpu().numpy()   # the generator's input (not a GPU result)
        xv = D.xv.cpu().numpy()
        y = D.y.cpu().numpy()
        errs = []
        for i in rows:
            a0, a1 = rp[i], rp[i + 1]
            ref = O.spmv_csr(np.array([0, a1 - a0], np.int32), col[a0:a1], val[a0:a1], xv)[0]
            errs.append(abs(y[i] - ref) / abs(ref) if ref else abs(y[i]))
        return {"max_rel_err": float(max(errs)), "ok": bool(max(errs) <= 1e-4), "tol": 1e-4,
                "sample": f"local rows {rows} (incl. the 3 heaviest)"}
    return None


# ------------------------------------------------------------------ GPU arm
def build_driver(a, X, dev):
    from paper_conf_asplos_lis0l0c17_b200 import drivers
    sz = sizes(a)
    if a.config == "atax":
        return drivers.AtaxFamily(sz["n"], X, dev)
    if a.config == "jacobi":
        return drivers.JacobiSlab(sz["side"], sz["side"], sz["iters"], X, dev, overlap=not a.no_overlap,
                                  halo=a.halo, fuse=jacobi_fuse(a), kernel=getattr(a, "jkernel", "tile"),
                                  tile_rows=getattr(a, "tile_rows", 0))
    if a.config in ("conv3", "conv7"):
        return drivers.ConvSlab(sz["side"], sz["side"], sz["R"], X, dev)
    return drivers.SpmvBlock(sz["scale"], X, dev, hot=a.hot)


def main():
    a = parse()
    if a.impl == "reference":
        return run_reference(a)
    import torch
    import torch.distributed as dist

    from paper_conf_asplos_lis0l0c17_b200 import drivers, ops

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if a.same_device:                 # test harness: every rank on GPU 0 (gloo exchanges), never a measurement
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if a.exchange == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    X = drivers.make_exchange(a.exchange, world, rank, local)
    dev = torch.device("cuda", local)
    D = build_driver(a, X, dev)
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    head = dict(HEADLINE[a.config])
    if a.backend:
        head["backend"] = a.backend
        if a.backend != "static":
            head.pop("num_clusters", None)
        if a.backend not in ("agent", "identity", "static"):
            head.pop("shub", None)                 # the shared-memory hub tier needs persistent agents
    if a.config == "jacobi" and a.jkernel == "tile" and not a.order:
        head["order"] = "row"
    if a.order:
        head["order"] = a.order
    for k, v in (("active_agents", a.active_agents), ("stages", a.stages), ("batch", a.batch)):
        if v:
            head[k] = v
    if a.staging != "default":
        head["staging"] = a.staging
    use_graph = a.config != "atax" and not a.no_graph     # atax: eager, per-kernel events

    def bar():
        if world > 1:
            dist.barrier()

    def maxr(v):
        if world > 1:
            t = torch.tensor([v], device=dev if dist.get_backend() == "nccl" else "cpu")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            return t.item()
        return v

    captured = [False]

    def timed(opts, steps, per_kernel=False):
        """(ms per step, per-kernel ms or None, launches in the timed region)"""
        if use_graph:
            D.graph = None
            captured[0] = bool(D.capture(opts))
        for _ in range(max(3, a.warmup)):
            D.step(opts)
        evs = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in range(steps)] \
            if per_kernel and a.config == "atax" else None
        t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        bar()
        torch.cuda.synchronize()
        n = 0
        t0.record(stream)
        for k in range(steps):
            n += D.step(opts, ev=evs[k]) if evs else D.step(opts)
        t1.record(stream)
        torch.cuda.synchronize()
        ms = maxr(t0.elapsed_time(t1)) / steps
        per = None
        if evs:
            per = {"atax": sum(e[0].elapsed_time(e[1]) for e in evs) / steps,
                   "bicg": sum(e[1].elapsed_time(e[2]) for e in evs) / steps,
                   "mvt": sum(e[2].elapsed_time(e[3]) for e in evs) / steps}
        if use_graph:
            D.graph = None
        return ms, per, n

    # -------- clustered (headline), then the comparators
    clocks = Clocks(local)
    ms_clu, per_clu, launches = timed(head, a.steps, per_kernel=True)
    clk = clocks.stop()
    head_captured = captured[0]
    cmp_steps = max(3, a.steps // 2)
    dflt = {"backend": "default"}
    ms_def_tma, per_def_tma, _ = timed(dict(dflt, staging="tma"), cmp_steps, per_kernel=True)
    ms_def_dir, per_def_dir = None, None
    if a.config != "spmv":
        ms_def_dir, per_def_dir, _ = timed(dict(dflt, staging="direct"), cmp_steps, per_kernel=True)
    if ms_def_dir is None or ms_def_tma <= ms_def_dir:
        ms_def, per_def, def_kind = ms_def_tma, per_def_tma, "tma-staged"
    else:
        ms_def, per_def, def_kind = ms_def_dir, per_def_dir, "direct-load"
    ms_id, _, _ = timed(identity_opts(head), cmp_steps)
    ms_tall = None
    if a.config == "jacobi" and getattr(D, "kname", "") == "jacobi5_wave" and world == 1:
        # context, not a comparator: the same wavefront kernel in hardware order on
        # 256-row logical CTAs (few restarts), the fastest Jacobi measured
        t0_, D.trows = D.trows, 256
        ms_tall, _, _ = timed(dict(dflt), cmp_steps)
        D.trows = t0_
    ms_two_pass = None
    if a.config == "atax" and D.fused_atax:         # the same clustered step with the two-pass ATAX
        D.fused_atax = False
        ms_two_pass, _, _ = timed(head, cmp_steps)
        D.fused_atax = True
    total_bytes = D.bytes_per_step()
    value = total_bytes / (ms_clu * 1e-3) / 1e9

    # -------- home fraction of the headline schedule (untimed launch with exec_sm)
    home = home_fraction(a, D, head, local) if world == 1 else None

    # -------- roofline of the dominant kernel
    pk = peaks()
    roof = roofline(a, D, head, ms_clu, per_clu, launches, clk, pk)

    # -------- e2e through the public API with host buffers (pinned), H2D / D2H inside
    e2e = None if a.no_e2e else e2e_run(a, D, head, stream, bar, maxr, total_bytes)

    # -------- oracle legs (rank 0): sampled parity, CPU baseline
    parity = None
    if not a.no_parity:
        if a.config == "atax":
            D.reset()
            D.step(head)
            torch.cuda.synchronize()
            if world > 1:                          # gather tmp (padded blocks) for the y = A^T tmp check
                spans = [shard_rows(D.m_total, world, g) for g in range(world)]
                cap = max(hi - lo for lo, hi in spans)
                send = torch.zeros(cap, device=dev)
                send[: D.m] = D.tmp
                recv = torch.zeros(cap * world, device=dev)
                X.allgather(send, recv)
                torch.cuda.synchronize()
                D.tmp_all = torch.cat([recv[g * cap: g * cap + (hi - lo)] for g, (lo, hi) in enumerate(spans)])
            else:
                D.tmp_all = D.tmp
        elif a.config == "jacobi":
            D.reset()
            D.step(head)
            torch.cuda.synchronize()
        if rank == 0:
            parity = parity_probe(a.config, D, world)
    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        g1, dt1, desc1, _ = oracle_sample(a.config, sizes(a), 8.0, omp=False)
        gN, dtN, descN, thr = oracle_sample(a.config, sizes(a), 8.0, omp=True)
        cpu = {"value": round(gN, 4), "unit": "GB/s", "cores": thr, "kind": "oracle",
               "sample": f"{descN} ({dtN:.1f} s, OpenMP build, {thr} threads)",
               "single_thread": {"value": round(g1, 4), "unit": "GB/s", "cores": 1,
                                 "sample": f"{desc1} ({dt1:.1f} s)"},
               "cpu": cpu_info()}

    live = None
    if rank == 0 and world == 1 and not a.no_ncu:
        live = live_ncu(a, head, "tma" if def_kind == "tma-staged" else "direct")
        if live and a.config == "atax" and roof.get("kernel", "").startswith("k_agent<GemvBody<32, 256, 1, 1>>"):
            pk_ = live["headline_per_kernel"].get("void k_agent<GemvBody<32, 256, 1, 1>>", {})
            if pk_:
                roof["traffic"] = (pk_.get("dram__bytes_read.sum", 0) + pk_.get("dram__bytes_write.sum", 0)) / 2
                roof["traffic_source"] = "ncu in this run (per launch, cold L2)"
        elif live and a.config != "atax":
            # scripts/ncu_step.py runs ONE launch's worth of Jacobi sweeps (iters = fuse), a whole step otherwise
            per = 1 if a.config == "jacobi" else max(1, roof.get("launches_per_step") or 1)
            roof["traffic"] = live["dram_bytes_per_step"]["headline"] / per
            roof["traffic_source"] = "ncu in this run (per launch, cold L2)"
            if a.config == "spmv":
                roof["request_roofs"] = request_roofs(live)
                for k, m in live["headline_per_kernel"].items():
                    if "Spmv" in k:
                        roof["traffic"] = m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
    if rank == 0:
        l2red, prof = l2_reductions(a.config, head)
        line = {"metric": METRIC, "value": round(value, 3), "unit": "GB/s", "n_gpus": world, "steps": a.steps,
                "warmup": max(3, a.warmup), "ms_per_step": round(ms_clu, 4), "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "f32",
                "data": "synthetic (counter-hash generators, generated on device)",
                "config": config_block(a, D, head, world, use_graph and head_captured),
                "speedup_vs_default": round(ms_def / ms_clu, 4),
                "speedup_vs_identity": round(ms_id / ms_clu, 4),
                "ms_per_step_default": round(ms_def, 4), "default_kind": def_kind,
                "ms_per_step_default_tma": round(ms_def_tma, 4),
                "ms_per_step_default_direct": None if ms_def_dir is None else round(ms_def_dir, 4),
                "ms_per_step_identity": round(ms_id, 4),
                "ms_per_step_default_256row_tiles": None if ms_tall is None else round(ms_tall, 4),
                "ms_per_step_two_pass_atax": None if ms_two_pass is None else round(ms_two_pass, 4),
                "roofline": roof, "clocks": clk, "e2e": e2e, "cpu_baseline": cpu, "gpu_launches": launches,
                "home_fraction": home, "parity": parity,
                "l2_sector_reduction": live if live else
                {"source": prof, "metric": "1 - lts__t_sectors_srcunit_tex(variant) / (reference order)", **l2red},
                "l2_sector_reduction_suite": {"source": prof, **l2red} if live else None}
        if a.config == "jacobi":
            line["sweeps_per_second"] = round(D.iters / (ms_clu * 1e-3), 1)
        if per_clu:
            line["per_kernel_ms"] = {k: round(v, 4) for k, v in per_clu.items()}
            line["per_kernel_ms_default"] = {k: round(v, 4) for k, v in per_def.items()}
        print(json.dumps(line), flush=True)
    if a.suite and rank == 0 and world == 1:
        import bench_suite
        bench_suite.run(a.suite)
    if world > 1:
        dist.destroy_process_group()
    return 0


def shard_rows(n, world, g):
    from paper_conf_asplos_lis0l0c17_b200 import shard
    return shard.row_range(n, world, g)


def config_block(a, D, head, world, use_graph):
    c = {"workload": WORKLOAD[a.config], **{k: v for k, v in head.items()}, "graph": use_graph,
         "parallelism": {"atax": f"row-shard x{world}", "jacobi": f"slab-shard x{world} (halo 1 row/sweep)",
                         "conv3": f"slab-shard x{world} (halo 1 row)", "conv7": f"slab-shard x{world} (halo 3 rows)",
                         "spmv": f"nnz-balanced row blocks x{world}"}[a.config]}
    if a.config == "atax":
        c.update(n=D.n, tile="32x256 (BICG, MVT); one row per logical CTA (one-pass ATAX)",
                 atax="one pass (CC_K_ATAX_FUSED)" if D.fused_atax else "two passes",
                 l2="inputs (1 GiB) larger than L2 (126 MB); no flush")
    elif a.config == "jacobi":
        wave = D.kname == "jacobi5_wave"
        c.update(rows=D.rows, cols=D.cols, iters=D.iters, sweeps_per_launch=D.fuse,
                 kernel="CC_K_JACOBI5_WAVE (strip wavefronts, R34)" if wave else "CC_K_JACOBI5 (tile-fused, R32)",
                 tile="64 rows x 120/112-column strips" if wave else "32x32",
                 launches=[list(c_) for c_ in D.calls()] if wave and D.x.world == 1 else None,
                 bytes="one read + one write of the field per launch (per sweep when unfused)",
                 overlap=getattr(D, "overlap", False), halo="fused LL (peer memory)" if D.fused else "exchange",
                 l2="2 x 1 GiB ping-pong buffers, larger than L2; no flush")
    elif a.config in ("conv3", "conv7"):
        c.update(rows=D.rows, cols=D.cols, R=D.R, tile="32x32",
                 l2="image 256 MiB in + 256 MiB out, larger than L2; no flush")
    else:
        c.update(rows=D.rows, nnz=D.nnz, hub_slots=D.A.n_hot,
                 l2="col/val 2 GiB larger than L2; x (64 MiB) fits, as it would in use")
    return c


SPMV_REQ_METRICS = ("l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed",
                    "lts__t_tag_requests.avg.pct_of_peak_sustained_elapsed",
                    "lts__t_tag_requests.max.pct_of_peak_sustained_elapsed")


def request_roofs(live):
    """SpMV: utilisation of the L1 -> L2 request port and of the L2 tag
    lookups (average and busiest slice) by the headline SpMV kernel, from the
    live ncu pass -- the roofs the gathers actually hit (one 32-byte sector per
    x gather), next to the HBM roofline the line reports."""
    for k, m in (live or {}).get("headline_per_kernel", {}).items():
        if "Spmv" in k and all(x in m for x in SPMV_REQ_METRICS):
            return {"kernel": k.replace("void ", ""), "unit": "% of peak sustained",
                    "l1_to_l2_request_port": round(m[SPMV_REQ_METRICS[0]], 2),
                    "l2_tag_lookups_avg": round(m[SPMV_REQ_METRICS[1]], 2),
                    "l2_tag_lookups_busiest_slice": round(m[SPMV_REQ_METRICS[2]], 2),
                    "source": "ncu in this run (scripts/ncu_step.py, one headline step)"}
    return None


def live_ncu(a, head, dflt_staging):
    """L2 sectors and DRAM bytes of one step of the headline schedule, default
    order and the identity control, measured in this run: scripts/ncu_step.py
    under `ncu --profile-from-start off --cache-control all` (a separate
    process, after the timed region; counts only, never a timing).  None when
    ncu is unavailable or fails."""
    import csv
    import io
    import shutil
    ncu = shutil.which("ncu") or ("/usr/local/cuda/bin/ncu" if os.path.exists("/usr/local/cuda/bin/ncu") else None)
    if not ncu:
        return None
    metrics = "lts__t_sectors_srcunit_tex.sum,dram__bytes_read.sum,dram__bytes_write.sum"
    if a.config == "spmv":                   # the request-side roofs of the gather-bound SpMV
        metrics += "," + ",".join(SPMV_REQ_METRICS)
    variants = {"headline": head, "default": dict(backend="default", staging=dflt_staging),
                "identity": identity_opts(head)}
    out = {}
    for name, opts in variants.items():
        cmd = [ncu, "--profile-from-start", "off", "--metrics", metrics, "--cache-control", "all",
               "--clock-control", "none", "--csv", sys.executable, os.path.join(ROOT, "scripts", "ncu_step.py"),
               "--config", a.config, "--opts", json.dumps(opts), "--hot", str(a.hot), "--fuse", str(jacobi_fuse(a)),
               "--jkernel", a.jkernel]
        if a.n:
            cmd += ["--size", str(a.n)]
        try:
            r = subprocess.run(cmd, capture_output=True, text=True, timeout=240)
        except Exception:
            return None
        rows = [row for row in csv.reader(io.StringIO(r.stdout)) if len(row) > 10]
        if not rows or rows[0][0] != "ID":
            return None
        h = rows[0]
        per_kernel, tot = {}, {}
        for row in rows[1:]:
            d = dict(zip(h, row))
            try:
                v = float(d["Metric Value"].replace(",", ""))
            except ValueError:
                continue
            m = d["Metric Name"]
            if "pct" not in m:                   # utilisations are per kernel, not additive
                tot[m] = tot.get(m, 0.0) + v
            k = d["Kernel Name"].split("(")[0]
            per_kernel.setdefault(k, {}).setdefault(m, 0.0)
            per_kernel[k][m] += v
        out[name] = {"l2_sectors": tot.get("lts__t_sectors_srcunit_tex.sum"),
                     "dram_bytes": tot.get("dram__bytes_read.sum", 0.0) + tot.get("dram__bytes_write.sum", 0.0),
                     "per_kernel": per_kernel}
    h, d, i = out["headline"], out["default"], out["identity"]
    return {"source": "ncu in this run (scripts/ncu_step.py, --cache-control all, one step per schedule"
                      + ("; jacobi: one launch of `fuse` sweeps" if a.config == "jacobi" else "") + ")",
            "metric": "1 - lts__t_sectors_srcunit_tex(headline step) / (reference step)",
            "vs_default_order": round(1 - h["l2_sectors"] / d["l2_sectors"], 4) if d["l2_sectors"] else None,
            "vs_identity_order": round(1 - h["l2_sectors"] / i["l2_sectors"], 4) if i["l2_sectors"] else None,
            "l2_sectors_per_step": {k: v["l2_sectors"] for k, v in out.items()},
            "dram_bytes_per_step": {k: v["dram_bytes"] for k, v in out.items()},
            "headline_per_kernel": h["per_kernel"]}


def l2_reductions(cfg, head):
    """L2-sector reductions vs default order and vs the identity (persistence
    only) order from the newest committed ncu summary (scripts/ncu_suite.sh);
    ncu cannot run inside this process."""
    import glob
    profs = sorted(glob.glob(os.path.join(ROOT, "profiles", "ncu_r*_summary.json")))
    if not profs:
        return {}, None
    try:
        pj = json.load(open(profs[-1]))
    except Exception:
        return {}, None
    kern = {"atax": ("atax", "bicg", "mvt"), "jacobi": ("jacobi",), "conv3": ("conv3",), "conv7": ("conv7",),
            "spmv": ("spmv",)}[cfg]
    rows = [r for r in pj.get("rows", []) if r.get("kernel") in kern]
    by = {(r["kernel"], r["variant"]): r for r in rows}
    vs_def, vs_id = {}, {}
    for (k, v), r in by.items():
        if r.get("l2_sm_sector_reduction_vs_default") is not None:
            vs_def[f"{k}:{v}"] = round(r["l2_sm_sector_reduction_vs_default"], 4)
        idr = by.get((k, "identity"))
        if idr and r.get("l2_sectors_sm") and idr.get("l2_sectors_sm") and v != "identity":
            vs_id[f"{k}:{v}"] = round(1 - r["l2_sectors_sm"] / idr["l2_sectors_sm"], 4)
    return {"vs_default_order": vs_def, "vs_identity_order": vs_id}, os.path.relpath(profs[-1], ROOT)


def identity_opts(head):
    """the persistence-only control of a headline schedule: the same body
    (SpMV's shared-memory hub tier included) in identity order"""
    return dict(backend="identity", **({"shub": True} if head.get("shub") else {}))


def roofline(a, D, head, ms_clu, per_clu, launches, clk, pk):
    peak_hbm = pk["hbm_gbs"] if pk else 6650.0
    src = "MEASURED_PEAKS.json hbm_gbs (copy)" if pk else "fallback 6.65 TB/s"
    traffic = traffic_from_profiles(a.config, head, a.hot)
    if a.config == "atax":
        from paper_conf_asplos_lis0l0c17_b200 import drivers
        b_local = drivers.atax_family_bytes(D.m, D.n)
        atax_fused = D.fused_atax and head.get("backend") in ("agent", "identity", "static")
        groups = {"gemv_fused": (("bicg", "mvt"), 2, "k_agent<GemvBody<32, 256, 1, 1>> (BICG, MVT)"),
                  "atax": (("atax",), 1, "k_agent<AtaxFusedBody> (one-pass ATAX)") if atax_fused else
                          (("atax",), 2, "k_agent<GemvBody<32, 256, 1, 0>> + <0, 1> (ATAX passes)")}
        gms = {g: sum(per_clu[k] for k in ks) for g, (ks, _, _) in groups.items()}
        dom = max(gms, key=gms.get)
        calls, nl, name = groups[dom]
        dbytes = sum(b_local[k] for k in calls) + (0 if atax_fused or dom != "atax" else 4 * D.m * D.n)
        ach = dbytes / (gms[dom] * 1e-3) / 1e9
        tr = None
        if traffic and all(traffic.get(k) for k in calls):
            tr = sum(traffic[k] for k in calls) / nl
        r = {"bound": "hbm", "kernel": name, "achieved": round(ach, 2), "peak": peak_hbm, "peak_source": src,
             "unit": "GB/s", "frac": round(ach / peak_hbm, 4), "traffic": tr, "launches_per_step": nl,
             "share_of_step": round(gms[dom] / sum(gms.values()), 4),
             "algorithmic_bytes_per_launch": dbytes // nl,
             "timing": "CUDA events around each kernel on the launching stream, mean over the timed steps",
             "frac_of_nominal_7700": round(ach / 7700.0, 4)}
        if ach > peak_hbm:
            r["note"] = ("the kernel streams A read-only (1 GiB read per launch, 0.1 % written); the measured "
                         "peak is a copy (half reads, half writes), which a read-only stream can exceed")
        return r
    # single-kernel configs: every launch in the step is the headline kernel
    # (SpMV's hub form adds one tiny hub-gather launch per step, 64 KB: it is
    # counted in the step time, not as a launch of the headline kernel)
    nl = max(1, launches // a.steps)
    if a.config == "spmv" and D.A.n_hot > 0:
        nl = max(1, nl - 1)
    ms_launch = ms_clu / nl
    if a.config == "jacobi" and D.kname == "jacobi5_wave":
        kind = {"agent": 0, "identity": 0, "static": 1, "default": 2}.get(head.get("backend"), 0)
        jk = f"k_strip<JwJacobi<{D.fuse}, {1 if D.fuse <= 4 else 2}>, {kind}>"
    body = {"jacobi": f"Jacobi5MultiBody<{D.fuse}>" if a.config == "jacobi" and D.fuse > 1 else "Jacobi5BodyT<false>",
            "conv3": "Conv2dBody<1>", "conv7": "Conv2dBody<3>",
            "spmv": "SpmvShubBody" if head.get("shub") else "SpmvBody"}[a.config]
    kern = {"agent": "k_agent", "static": "k_static", "default": "k_default", "identity": "k_agent"}.get(
        head.get("backend"), "k_agent") + f"<{body}>"
    if a.config == "jacobi" and D.kname == "jacobi5_wave":
        kern = jk
    bpl = D.bytes_per_step() // nl if D.x.world == 1 else None
    tr = traffic.get(a.config) if traffic else None
    if a.config == "conv7":
        mhz = clk.get("sm_mhz") or 1965.0
        peak = NSM * 128 * 2 * mhz * 1e6 / 1e12
        fl = D.flops_per_step() / nl
        ach = fl / (ms_launch * 1e-3) / 1e12
        return {"bound": "alu", "kernel": kern, "achieved": round(ach, 2), "peak": round(peak, 2), "unit": "TFLOP/s",
                "frac": round(ach / peak, 4), "peak_source": f"148 SM x 128 FP32 FMA/clk x 2 x {mhz:.0f} MHz "
                                                             "(median SM clock under load)",
                "traffic": tr, "launches_per_step": nl, "share_of_step": 1.0,
                "algorithmic_flops_per_launch": fl, "algorithmic_bytes_per_launch": bpl,
                "timing": "step time / launches (one kernel per step)"}
    ach = (D.bytes_per_step() / nl) / (ms_launch * 1e-3) / 1e9
    r = {"bound": "hbm", "kernel": kern, "achieved": round(ach, 2), "peak": peak_hbm, "peak_source": src,
         "unit": "GB/s", "frac": round(ach / peak_hbm, 4), "traffic": tr, "launches_per_step": nl,
         "share_of_step": 1.0 if D.x.world == 1 else None, "algorithmic_bytes_per_launch": bpl,
         "timing": "step time / launches: the step is back-to-back launches of this one kernel"
                   + (" (whole-job bytes, includes the exchange at N > 1)" if D.x.world > 1 else "")}
    if a.config == "jacobi" and D.kname == "jacobi5_wave" and D.x.world == 1:
        # K sweeps per read + write of the field: the second roof is the FP32
        # pipe -- 5 FP32 instructions (4 FADD + FMUL, PolyBench order, no FMA)
        # per point and sweep against 148 SM x 128 lanes x the SM clock
        mhz = clk.get("sm_mhz") or 1965.0
        peak_fp = NSM * 128 * mhz * 1e6 / 1e12
        fp = 5.0 * D.rows * D.cols * D.iters / (ms_clu * 1e-3) / 1e12
        r["alu"] = {"achieved": round(fp, 2), "peak": round(peak_fp, 2), "frac": round(fp / peak_fp, 4),
                    "unit": "T FP32 instructions/s",
                    "peak_source": f"148 SM x 128 FP32 lanes x {mhz:.0f} MHz (median SM clock under load)",
                    "note": "issue-bound between the two roofs: ~270 instructions per row step of 8 levels, "
                            "176 of them FP32 + shuffles (ncu, profiles/final)"}
    return r


def traffic_from_profiles(cfg, head, hot=0):
    """ncu dram bytes per launch of the headline variant from the newest
    committed summary (cold-cache, one launch)."""
    import glob
    profs = sorted(glob.glob(os.path.join(ROOT, "profiles", "ncu_r*_summary.json")))
    if not profs:
        return None
    try:
        d = json.load(open(profs[-1])).get("dram_bytes_per_launch", {})
    except Exception:
        return None
    b, o = head.get("backend"), head.get("order")
    suf = b + (f"-{o}" if o and b in ("agent", "static") else "")
    if b == "static" and head.get("num_clusters"):
        suf += f"-m{head['num_clusters'] // NSM}"
    out = {}
    for k in ("atax", "bicg", "mvt", "jacobi", "conv3", "conv7", "spmv"):
        if f"{k}_{suf}" in d:
            out[k] = d[f"{k}_{suf}"]
    if cfg == "spmv" and hot and f"spmv_{suf}-hot" in d:        # the hub-column form's capture
        out["spmv"] = d[f"spmv_{suf}-hot"]
    return out


def home_fraction(a, D, head, device):
    """Share of logical CTAs executed on their home SM (the SM of dense rank i
    for cluster i) in one untimed launch of the headline schedule with exec_sm
    recording (stealing on)."""
    import numpy as np
    import torch
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    if head.get("backend") not in ("agent", "static"):
        return None
    try:
        if a.config == "atax":
            args = cc.bicg_args(D.A, D.p, D.r, D.q, D.s)
            kern = "bicg"
        elif a.config == "jacobi":
            args = cc.jacobi5_args(D.a, D.b, D.fuse, fuse=D.fuse)[0]       # one launch of the headline kernel
            kern = D.kname
        elif a.config in ("conv3", "conv7"):
            args, D._w = cc.conv2d_args(D.inp, D.out, D.w)
            kern = "conv2d"
        else:
            args = D.A.args(D.xv, D.y)
            kern = "spmv_shub" if head.get("shub") else "spmv"
        kw = dict(head)
        kw.pop("shub", None)
        order, nc = kw.pop("order", None), kw.pop("num_clusters", 0)
        from paper_conf_asplos_lis0l0c17_b200 import ops
        p = ops.plan_for(kern, args, order, kw.pop("tile", None), nc, device)
        V = p.V
        sm = torch.full((V,), -1, dtype=torch.int32, device="cuda")
        cc.launch(p, kern, args, cc.make_opts(exec_sm=sm, **kw))
        torch.cuda.synchronize()
        perm, off = p.table()
        rank_of = cc.sm_rank_table(device)
        smv = sm.cpu().numpy()
        rank_exec = np.where(smv >= 0, rank_of[np.clip(smv, 0, len(rank_of) - 1)], -1)
        cluster = np.empty(V, np.int64)
        cluster[perm] = np.repeat(np.arange(p.M), np.diff(off))
        if head.get("backend") == "static":
            # static binding: cluster i is one CTA; "home" = all of a cluster on one SM
            same = [len(set(smv[perm[off[i]:off[i + 1]]])) <= 1 for i in range(p.M)]
            return {"value": round(float(np.mean(same)), 4), "kind": "clusters executed on one SM (static binding)"}
        home = cluster % NSM if p.M > NSM else cluster
        return {"value": round(float(np.mean(rank_exec == home)), 4),
                "kind": "tasks run on their cluster's home SM (stealing on)", "launch": kern}
    except Exception as e:
        return {"error": repr(e)[:200]}


def e2e_run(a, D, head, stream, bar, maxr, total_bytes):
    """The same metric through the public API with the step's inputs copied
    from pinned host memory and its outputs read back, inside the timed region."""
    import torch
    if a.config == "atax":
        ins, outs = D.inputs(), D.outputs()
    elif a.config == "jacobi":
        ins, outs = {"u": D.a}, {"u": D.a}
    elif a.config in ("conv3", "conv7"):
        ins, outs = {"inp": D.inp}, {"out": D.out}
    else:
        Am = D.A
        ins = {"row_ptr": Am.row_ptr, "col": Am.col_kernel, "val": Am.val, "x": D.xv}
        if Am.hot is not None:
            ins["hot"] = Am.hot
        outs = {"y": D.y}
    h_in = {k: v.cpu().pin_memory() for k, v in ins.items()}
    h_out = {k: torch.empty(v.shape, dtype=v.dtype, pin_memory=True) for k, v in outs.items()}

    def step():
        for k, t_ in ins.items():
            t_.copy_(h_in[k], non_blocking=True)
        D.step(head)
        for k, t_ in outs.items():
            h_out[k].copy_(t_, non_blocking=True)
    steps = max(3, min(10, a.steps))
    if a.config == "jacobi":
        D.graph = None
        steps = 3
    step()
    torch.cuda.synchronize()
    bar()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0.record(stream)
    for _ in range(steps):
        step()
    t1.record(stream)
    torch.cuda.synchronize()
    ms = maxr(t0.elapsed_time(t1) / steps)
    h2d = sum(v.numel() * v.element_size() for v in h_in.values())
    d2h = sum(v.numel() * v.element_size() for v in h_out.values())
    return {"value": round(total_bytes / (ms * 1e-3) / 1e9, 3), "unit": "GB/s", "ms_per_step": round(ms, 3),
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h}


if __name__ == "__main__":
    sys.exit(main())
