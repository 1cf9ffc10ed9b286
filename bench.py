#!/usr/bin/env python
"""bench.py -- BASELINE config 2 on B200: PolyBench ATAX + BICG + MVT, fp32,
n = 16384, column clustering (the paper's X-partition for ATX/MVT/BC, Table 2
P:2297-2301) with the agent runtime, row-sharded over N GPUs.

One step = ATAX (2 passes) + BICG (1 fused pass) + MVT (1 fused pass) over the
1 GiB matrix: four streaming passes, HBM-bound.  `value` is algorithmic HBM
bytes per second (whole job); the same step under the default hardware CTA
order is timed back to back and reported as `speedup_vs_default`.

    python bench.py [--gpus N --steps K --warmup W] [--impl reference] [--suite out.json]

Rules kept: W >= 3 warm-ups; K timed steps bracketed by barrier + synchronize,
CUDA events on the launching stream, max over ranks; the matrix (1 GiB) is
larger than L2 (126 MB) so no flush is needed; nvidia-smi clocks sampled during
the timed region.  The oracle (oracle/, CPU) is only run in the cpu_baseline
leg and in --impl reference.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "speedup & L2 sector reduction vs default CTA order; HBM GB/s vs roofline"
N_DIM = 16384


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", type=int, default=N_DIM)
    ap.add_argument("--backend", default="agent")
    ap.add_argument("--order", default="col")
    ap.add_argument("--active-agents", type=int, default=0)
    ap.add_argument("--stages", type=int, default=0)
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--staging", default="default", choices=["default", "tma", "direct"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--suite", default=None, help="also run every BASELINE config, write JSON here")
    return ap.parse_args()


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return None


def step_bytes(m, n):
    """Algorithmic bytes of one step (each pass reads A once; vectors once;
    outputs written once; MVT's x1/x2 read and written)."""
    A = 4 * m * n
    atax = (A + 4 * n + 4 * m) + (A + 4 * m + 4 * n)
    bicg = A + 4 * (n + m) + 4 * (m + n)
    mvt = A + 4 * (n + m) + 8 * (m + n)
    return {"atax": atax, "bicg": bicg, "mvt": mvt, "total": atax + bicg + mvt}


# ------------------------------------------------------------------ clocks
class Clocks:
    def __init__(self, device_index):
        self.p = None
        self.path = os.path.join("/tmp", f"cc_clocks_{os.getpid()}.csv")
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.f = open(self.path, "w")
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(device_index), f"--query-gpu={q}",
                                       "--format=csv,noheader,nounits", "-lms", "20"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.close()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in open(self.path):
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        os.unlink(self.path)
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "samples": len(sm), "reasons": sorted(reasons)}


# ------------------------------------------------------------------ oracle legs
def oracle_sample(rows, n, reps, min_secs=0.0):
    """The oracle (plain C, fp64, one thread) on rows [0, rows) of the same A:
    ATAX + BICG + MVT, `reps` times and then on until `min_secs` have passed.
    Returns (GB/s in the metric's algorithmic bytes, secs, reps run)."""
    import numpy as np
    import oracle as O
    from paper_conf_asplos_lis0l0c17_b200 import synth
    A = synth.matrix(3, rows, n)
    x, p = synth.uniform(10, n), synth.uniform(11, n)
    r, x1 = synth.uniform(12, rows), synth.uniform(13, rows)
    x2, y1, y2 = synth.uniform(14, n), synth.uniform(15, n), synth.uniform(16, rows)
    t0 = time.perf_counter()
    done = 0
    while done < reps or time.perf_counter() - t0 < min_secs:
        O.atax(A, x)
        O.bicg(A, p, r)
        O.mvt(A, x1, x2, y1, y2)
        done += 1
    dt = time.perf_counter() - t0
    return done * step_bytes(rows, n)["total"] / dt / 1e9, dt, done


def run_reference(a):
    import torch.distributed as dist
    rank = int(os.environ.get("RANK", "0"))
    if int(os.environ.get("WORLD_SIZE", "1")) > 1 and rank != 0:
        return 0
    rows = 2048
    for _ in range(max(0, a.warmup)):
        oracle_sample(256, a.n, 1)
    gbs, dt, _ = oracle_sample(rows, a.n, a.steps)
    line = {"impl": "reference", "metric": METRIC, "value": round(gbs, 4), "unit": "GB/s", "n_gpus": a.gpus,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": round(1e3 * dt / a.steps, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (counter-hash U[0,1), seed 3)",
            "config": {"workload": f"ATAX+BICG+MVT fp32 n={a.n} (BASELINE config 2)",
                       "sample": f"rows 0..{rows - 1} per step (oracle, fp64, one host thread)"},
            "cpu_baseline": {"value": round(gbs, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": f"ATAX+BICG+MVT on rows 0..{rows - 1} of the {a.n}x{a.n} matrix, per step"},
            "e2e": {"value": round(gbs, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ GPU arm
def main():
    a = parse()
    if a.impl == "reference":
        return run_reference(a)
    import torch
    import torch.distributed as dist

    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, shard, synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    comm = None
    if world > 1:
        # the library's own NCCL communicator (cc_comm_*); torch.distributed only
        # carries the unique id
        box = [cc.Comm.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(box, src=0)
        comm = cc.Comm(box[0], world, rank, local)
    dev = torch.device("cuda", local)
    n = a.n
    lo, hi = shard.row_range(n, world, rank)
    m = hi - lo
    stream = torch.cuda.current_stream()

    # inputs: generated in place on the device by the shared counter-hash generator
    A = synth.matrix(3, m, n, backend="torch", device=dev, row0=lo)
    col = lambda seed: synth.uniform(seed, n, backend="torch", device=dev)
    row = lambda seed: synth.uniform(seed, m, lo, backend="torch", device=dev)
    x, p, y1 = col(10), col(11), col(15)
    r, x1_0, y2 = row(12), row(13), row(16)
    x2_0 = col(14)
    # the three column-indexed (transposed-product) outputs live in one buffer
    # so that N > 1 sums them over the ranks with a single all-reduce per step
    tsum = torch.empty(3 * n, device=dev)
    y, s, x2 = tsum[:n], tsum[n:2 * n], tsum[2 * n:]
    tmp, q = torch.empty(m, device=dev), torch.empty(m, device=dev)
    x1 = x1_0.clone()
    x2.copy_(x2_0 if rank == 0 else torch.zeros(n, device=dev))
    torch.cuda.synchronize()

    def run_step(backend, order, ev=None, count=None, staging=None):
        kw = dict(backend=backend, active_agents=a.active_agents, stages=a.stages, batch=a.batch,
                  staging=a.staging if staging is None else staging)
        nl = 0
        if ev is not None: ev[0].record(stream)
        pl = ops.plan_for("atax", cc.atax_args(A, x, tmp, y), order)
        nl += cc.launch(pl, "atax", cc.atax_args(A, x, tmp, y), cc.make_opts(**kw), stream)
        if ev is not None: ev[1].record(stream)
        nl += cc.launch(pl, "bicg", cc.bicg_args(A, p, r, q, s), cc.make_opts(**kw), stream)
        if ev is not None: ev[2].record(stream)
        nl += cc.launch(pl, "mvt", cc.mvt_args(A, y1, y2, x1, x2), cc.make_opts(**kw), stream)
        if ev is not None: ev[3].record(stream)
        if world > 1:                                # transposed products: one sum over ranks
            comm.allreduce_sum(tsum, stream)
        if count is not None:
            count[0] += nl

    def timed(backend, order, steps, per_kernel=False, staging=None):
        for _ in range(max(3, a.warmup)):
            run_step(backend, order, staging=staging)
        evs = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in range(steps)] if per_kernel else None
        t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        count = [0]
        t0.record(stream)
        for k in range(steps):
            run_step(backend, order, evs[k] if evs else None, count, staging)
        t1.record(stream)
        torch.cuda.synchronize()
        ms = t0.elapsed_time(t1)
        if world > 1:
            tt = torch.tensor([ms], device=dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ms = tt.item()
        per = None
        if evs:
            per = {"atax": sum(e[0].elapsed_time(e[1]) for e in evs) / steps,
                   "bicg": sum(e[1].elapsed_time(e[2]) for e in evs) / steps,
                   "mvt": sum(e[2].elapsed_time(e[3]) for e in evs) / steps}
        return ms / steps, per, count[0]

    # -------- clustered (headline) and default-order comparator
    clocks = Clocks(local)
    ms_clu, per_clu, launches = timed(a.backend, a.order, a.steps, per_kernel=True)
    clk = clocks.stop()
    # default hardware CTA order: the same TMA-staged body, and the plain
    # direct-load kernel; the faster one is the comparator
    ms_def_tma, per_def_tma, _ = timed("default", "row", a.steps, per_kernel=True, staging="tma")
    ms_def_dir, per_def_dir, _ = timed("default", "row", a.steps, per_kernel=True, staging="direct")
    ms_def, per_def, def_kind = ((ms_def_tma, per_def_tma, "tma-staged") if ms_def_tma <= ms_def_dir
                                 else (ms_def_dir, per_def_dir, "direct-load"))
    ms_id, _, _ = timed("identity", "row", max(20, a.steps // 5))
    bytes_all = step_bytes(n, n)              # whole job: every rank's rows together
    value = bytes_all["total"] / (ms_clu * 1e-3) / 1e9

    # -------- roofline of the dominant kernel (largest share of the step)
    pk = peaks()
    peak = pk["hbm_gbs"] if pk else 6650.0
    # kernels = instantiations in the launch list: the fused row+column gemv
    # (GemvBody<32,256,1,1>) runs BICG and MVT; ATAX is two single-direction
    # passes (<1,0>, <0,1>).  The dominant one is the largest share of the step.
    b_local = step_bytes(m, n)
    groups = {"gemv_fused": (("bicg", "mvt"), 2, "k_agent<GemvBody<32, 256, 1, 1>> (BICG, MVT)"),
              "atax": (("atax",), 2, "k_agent<GemvBody<32, 256, 1, 0>> + <0, 1> (ATAX passes)")}
    gms = {g: sum(per_clu[k] for k in ks) for g, (ks, _, _) in groups.items()}
    dom = max(gms, key=gms.get)
    dom_calls, dom_launches, dom_name = groups[dom]
    dom_bytes = sum(b_local[k] for k in dom_calls)
    achieved = dom_bytes / (gms[dom] * 1e-3) / 1e9        # = bytes per launch / mean launch time
    # DRAM bytes per launch of that kernel from the newest committed ncu capture
    # (profiles/ncu_<round>_summary.json, scripts/ncu_suite.sh); the L2-sector
    # reduction vs default order comes from the same capture.
    traffic, l2red, prof_name = None, None, None
    import glob
    profs = sorted(glob.glob(os.path.join(ROOT, "profiles", "ncu_r*_summary.json")))
    if profs:
        try:
            pj = json.load(open(profs[-1]))
            prof_name = os.path.relpath(profs[-1], ROOT)
            suf = f"_{a.backend}-{a.order}" + ("" if a.staging in ("default", "tma") else f"-{a.staging}")
            per_l = [pj.get("dram_bytes_per_launch", {}).get(k + suf) for k in dom_calls]
            if all(t_ is not None for t_ in per_l):     # the ATAX entry covers its two launches
                traffic = sum(per_l) / dom_launches
            l2red = {f"{r['kernel']}:{r['variant']}": round(r["l2_sm_sector_reduction_vs_default"], 4)
                     for r in pj.get("rows", []) if r.get("l2_sm_sector_reduction_vs_default") is not None
                     and r["kernel"] in ("atax", "bicg", "mvt")}
        except Exception:
            traffic = None

    # -------- e2e through the public API with host buffers (pinned), H2D/D2H inside
    e2e = None
    if not a.no_e2e:
        hA = A.cpu().pin_memory()
        hv = {k: v.cpu().pin_memory() for k, v in dict(x=x, p=p, r=r, y1=y1, y2=y2, x1=x1_0, x2=x2_0).items()}
        outs = {k: torch.empty(v.numel(), pin_memory=True) for k, v in dict(tmp=tmp, y=y, q=q, s=s, x1=x1, x2=x2).items()}
        e_steps = max(3, min(10, a.steps))

        def e2e_step():
            A.copy_(hA, non_blocking=True)
            for k, t_ in dict(x=x, p=p, r=r, y1=y1, y2=y2, x1=x1, x2=x2).items():
                t_.copy_(hv[k], non_blocking=True)
            run_step(a.backend, a.order)
            for k, t_ in dict(tmp=tmp, y=y, q=q, s=s, x1=x1, x2=x2).items():
                outs[k].copy_(t_, non_blocking=True)
        e2e_step()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for _ in range(e_steps):
            e2e_step()
        t1.record(stream)
        torch.cuda.synchronize()
        ems = t0.elapsed_time(t1) / e_steps
        if world > 1:
            tt = torch.tensor([ems], device=dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ems = tt.item()
        h2d = hA.numel() * 4 + sum(v.numel() * 4 for v in hv.values())
        d2h = sum(v.numel() * 4 for v in outs.values())
        e2e = {"value": round(bytes_all["total"] / (ems * 1e-3) / 1e9, 3), "unit": "GB/s",
               "ms_per_step": round(ems, 3), "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h}

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        # bounded sample: rows 0..4095 of the same matrix, repeated for >= 10 s
        gbs, dt, reps = oracle_sample(4096, n, 2, min_secs=10.0)
        cpu = {"value": round(gbs, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"ATAX+BICG+MVT on rows 0..4095 of the {n}x{n} matrix x{reps} reps ({dt:.1f} s)"}

    if rank == 0:
        line = {"metric": METRIC, "value": round(value, 3), "unit": "GB/s", "n_gpus": world, "steps": a.steps,
                "warmup": max(3, a.warmup), "ms_per_step": round(ms_clu, 4), "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "f32",
                "data": "synthetic (counter-hash U[0,1), generated on device)",
                "config": {"workload": f"ATAX+BICG+MVT fp32 n={n} (BASELINE config 2)",
                           "backend": a.backend, "order": a.order, "active_agents": a.active_agents or "max",
                           "stages": a.stages or "default", "batch": a.batch or "default", "staging": a.staging,
                           "tile": "32x256", "parallelism": f"row-shard x{world}",
                           "l2": "inputs (1 GiB) larger than L2 (126 MB); no flush"},
                "speedup_vs_default": round(ms_def / ms_clu, 4),
                "ms_per_step_default": round(ms_def, 4), "default_kind": def_kind,
                "ms_per_step_default_tma": round(ms_def_tma, 4), "ms_per_step_default_direct": round(ms_def_dir, 4),
                "ms_per_step_identity": round(ms_id, 4),
                "per_kernel_ms": {k: round(v, 4) for k, v in per_clu.items()},
                "per_kernel_ms_default": {k: round(v, 4) for k, v in per_def.items()},
                "roofline": {"bound": "hbm", "kernel": dom_name, "achieved": round(achieved, 2),
                             "peak": peak, "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy)" if pk else "fallback 6.65 TB/s",
                             "unit": "GB/s", "frac": round(achieved / peak, 4), "traffic": traffic,
                             "launches_per_step": dom_launches, "share_of_step": round(gms[dom] / sum(gms.values()), 4),
                             "algorithmic_bytes_per_launch": dom_bytes // dom_launches,
                             "note": "peak is the copy (read+write) figure while these kernels stream reads of A; "
                                     "traffic is ncu's cold-cache DRAM bytes per launch"},
                "clocks": clk, "e2e": e2e, "cpu_baseline": cpu, "gpu_launches": launches,
                "l2_sector_reduction": {"source": prof_name, "vs_default_order": l2red,
                                        "metric": "1 - lts__t_sectors_srcunit_tex(variant) / (default order)"}}
        print(json.dumps(line), flush=True)
    if a.suite and rank == 0 and world == 1:
        import bench_suite
        bench_suite.run(a.suite)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
