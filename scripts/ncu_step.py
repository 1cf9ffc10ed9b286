#!/usr/bin/env python
"""One bench step of a config under a given schedule, bracketed by
cudaProfilerStart / Stop, for `ncu --profile-from-start off` (bench.py runs it
to measure L2 sectors and DRAM bytes of the timed schedules live).

    python scripts/ncu_step.py --config atax --backend agent --order col
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="atax")
    ap.add_argument("--opts", default="{}", help="launch options as JSON (bench HEADLINE form)")
    ap.add_argument("--size", type=int, default=0)
    ap.add_argument("--hot", type=int, default=16384)
    ap.add_argument("--fuse", type=int, default=3)
    ap.add_argument("--jkernel", default="tile")
    a = ap.parse_args()
    import torch
    import bench
    from paper_conf_asplos_lis0l0c17_b200 import drivers
    ns = argparse.Namespace(config=a.config, n=a.size, iters=100, no_overlap=True, halo="exchange", fuse=a.fuse,
                            hot=a.hot, jkernel=a.jkernel)
    D = bench.build_driver(ns, drivers.Exchange(), torch.device("cuda", 0))
    opts = json.loads(a.opts)
    if a.config == "jacobi":                   # one launch's worth of sweeps is enough for per-launch counts
        D.iters = D.fuse if D.fuse > 1 else 1
    D.step(opts)                               # warm-up: plans, tensor maps
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    n = D.step(opts)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print(json.dumps({"launches": n}), flush=True)


if __name__ == "__main__":
    main()
