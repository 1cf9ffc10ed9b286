#!/usr/bin/env python
"""Column-strip wavefront Jacobi (CC_K_JACOBI5_WAVE, reading R34) vs the
tile-fused sweeps (CC_K_JACOBI5, fuse = 3, the round-2 bench default):
100 sweeps of the 16384^2 field, graph-timed (one graph per variant).
    python scripts/exp_jwave.py out.json [fuse,fuse,...]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench_suite as B  # noqa: E402


def main():
    import numpy as np
    import torch
    import oracle as O
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, synth
    fuses = [int(f) for f in sys.argv[2].split(",")] if len(sys.argv) > 2 else [2, 3, 4, 5, 6, 8]
    # quick parity gate before timing
    u0 = synth.matrix(7, 517, 388)
    a = torch.from_numpy(u0).cuda()
    for f in fuses:
        for v in (dict(backend="agent", order="col"), dict(backend="identity"), dict(backend="default")):
            got = ops.jacobi5_wave(a.clone(), torch.empty_like(a), 2 * f + 1, fuse=f, **v)
            assert np.array_equal(got.cpu().numpy(), O.jacobi5_f32(u0, 2 * f + 1)), (f, v)
    print("parity ok", flush=True)
    N, T = 16384, 100
    a = synth.matrix(4, N, N, backend="torch", device="cuda")
    b = a.clone()
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    rows = []

    def timed(name, fn, extra):
        ms = B.graph_ms(fn, 3, 1)
        r = {"variant": name, "ms_per_100_sweeps": round(ms, 3), **extra}
        rows.append(r)
        print(r, flush=True)

    timed("tilefused3-agent-row", lambda: ops.jacobi5(a, b, T, fuse=3, backend="agent", order="row"), {})
    timed("tilefused3-identity", lambda: ops.jacobi5(a, b, T, fuse=3, backend="identity"), {})
    for f in fuses:
        wpsm = cc.max_agents("jacobi5_wave", 0) if f <= 4 else None
        launches = -(-T // f)
        base = {"fuse": f, "launches": launches, "hbm_floor_ms": round(launches * 8 * N * N / B._peak() / 1e6, 3)}
        extra = []
        if os.environ.get("JW_HINTS"):
            extra = [(f"{b}-{h}", dict(backend=b, l2_hint=h, **({"order": "col"} if b == "agent" else {})))
                     for b in ("agent", "default") for h in ("stream_first", "reuse_last", "both")]
        for name, kw in extra + [("agent-col", dict(backend="agent", order="col")),
                         ("agent-col-b8", dict(backend="agent", order="col", batch=8)),
                         ("agent-col-b4", dict(backend="agent", order="col", batch=4)),
                         ("agent-col-b2", dict(backend="agent", order="col", batch=2)),
                         ("agent-col-b1", dict(backend="agent", order="col", batch=1)),
                         ("static-col", dict(backend="static", order="col", num_clusters=sms * (24 if f <= 3 else 20 if f == 4 else 15))),
                         ("agent-row", dict(backend="agent", order="row")),
                         ("static-tile1x16", dict(backend="static", order="tile", tile=(1, 16),
                                                  num_clusters=-(-(-(-N // (128 - 8 * (1 if f <= 4 else 2)))) * (N // 64) // 16))),
                         ("static-tile1x8", dict(backend="static", order="tile", tile=(1, 8),
                                                 num_clusters=-(-(-(-N // (128 - 8 * (1 if f <= 4 else 2)))) * (N // 64) // 8))),
                         ("agent-tile1x16-b16", dict(backend="agent", order="tile", tile=(1, 16), batch=16)),
                         ("agent-tile1x8-b8", dict(backend="agent", order="tile", tile=(1, 8), batch=8)),
                         ("identity", dict(backend="identity")),
                         ("default", dict(backend="default"))]:
            kw = dict(kw, tile_rows=int(os.environ.get("JW_TROWS", "0")))
            timed(f"wave{f}-{name}", lambda kw=kw, f=f: ops.jacobi5_wave(a, b, T, fuse=f, **kw),
                  dict(base, warps_per_sm=wpsm))
    json.dump({"N": N, "sweeps": T, "rows": rows}, open(sys.argv[1], "w"), indent=1)


if __name__ == "__main__":
    main()
