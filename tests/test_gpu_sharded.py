"""GPU parity of the sharded drivers (drivers.py, S§8(e)) -- VERDICT r1 item 2.

The N > 1 CUDA path runs here as G ranks in G processes sharing one GPU
(gloo carries the exchanges, staged through host memory; on a multi-GPU box
the same drivers use the library's NCCL communicator).  Every rank's shard
runs the library's kernels; the combined result must equal the unsharded
oracle: bit for bit for Jacobi (fp32 oracle, same order per point), <= 1e-4
relative otherwise (positive inputs, C17).  The row-window form of the Jacobi
sweep that the boundary-first overlap relies on is checked on its own.
"""
import os
import socket
import subprocess
import sys
import textwrap

import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_asplos_lis0l0c17_b200 import drivers, ops, synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def rel(got, ref):
    got = np.asarray(got, dtype=np.float64)
    return float(np.max(np.abs(got - ref) / np.abs(ref))) if ref.size else 0.0


# ---------------------------------------------------------------- row windows
def padded(u0, fill=0.0):
    """device copy with a 16-byte leading dimension (ragged widths keep ld % 4 == 0)"""
    rows, cols = u0.shape
    t = torch.full((rows, (cols + 3) & ~3), fill, device="cuda")[:, :cols]
    t.copy_(torch.from_numpy(np.ascontiguousarray(u0)))
    return t


@pytest.mark.parametrize("backend,order", [("agent", "row"), ("default", None), ("identity", None),
                                           ("static", "row"), ("agent", "tile")])
@pytest.mark.parametrize("rows,cols,win", [(130, 100, (1, 33)), (130, 100, (33, 97)), (130, 100, (97, 130)),
                                            (130, 100, (0, 130)), (77, 45, (5, 6)), (77, 45, (0, 40))])
def test_jacobi_row_window(backend, order, rows, cols, win):
    u0 = synth.matrix(4, rows, cols)
    a = padded(u0)
    sentinel = np.float32(-7.0)
    b = padded(np.full_like(u0, sentinel))
    kw = dict(backend=backend)
    if order:
        kw["order"] = order
    if order == "tile":
        kw["tile"] = (2, 2)
    ops.jacobi5(a, b, 1, row_window=win, **kw)
    torch.cuda.synchronize()
    got = b.cpu().numpy()
    ref = O.jacobi5_f32(u0, 1)
    lo, hi = win
    assert np.array_equal(got[lo:hi], ref[lo:hi])
    outside = np.concatenate([got[:lo], got[hi:]])
    assert np.all(outside == sentinel)


def test_jacobi_windows_compose_to_full_sweep():
    """boundary windows + interior window = the full sweep, several sweeps"""
    rows, cols, T = 200, 130, 5
    u0 = synth.matrix(4, rows, cols)
    a = padded(u0)
    b = padded(u0)
    wins = [(0, 32), (168, 200), (32, 168)]
    for k in range(T):
        src, dst = (a, b) if k % 2 == 0 else (b, a)
        for w in wins:
            ops.jacobi5(src, dst, 1, row_window=w, backend="agent", order="row")
    torch.cuda.synchronize()
    out = (b if T % 2 else a).cpu().numpy()
    assert np.array_equal(out, O.jacobi5_f32(u0, T))


def test_jacobi_window_errors():
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    a = torch.zeros(64, 64, device="cuda")
    for w in [(10, 5), (-1, 3), (0, 65)]:
        with pytest.raises(cc.CtaclustError):
            ops.jacobi5(a, a.clone(), 1, row_window=w)


# ---------------------------------------------------------------- world = 1 drivers
def test_atax_family_driver_world1():
    n = 700
    d = drivers.AtaxFamily(n, drivers.Exchange(), "cuda")
    d.step(dict(backend="agent", order="col"))
    torch.cuda.synchronize()
    A = synth.matrix(3, n, n)
    x, p, r = synth.uniform(10, n), synth.uniform(11, n), synth.uniform(12, n)
    x1, x2, y1, y2 = synth.uniform(13, n), synth.uniform(14, n), synth.uniform(15, n), synth.uniform(16, n)
    tmp, y = O.atax(A, x)
    q, s = O.bicg(A, p, r)
    o1, o2 = O.mvt(A, x1, x2, y1, y2)
    for got, ref in ((d.tmp, tmp), (d.y, y), (d.q, q), (d.s, s), (d.x1, o1), (d.x2, o2)):
        assert rel(got.cpu().numpy(), ref) <= 1e-4


@pytest.mark.parametrize("fuse,T", [(8, 100), (8, 13), (3, 7), (6, 20), (8, 16)])
def test_jacobi_wave_driver_world1_graph(fuse, T):
    """The bench's config-3 driver with the wavefront kernel, captured and
    replayed (an odd launch count ends in the other buffer: two graphs, one
    from each buffer, alternate), bit-exact over three consecutive steps."""
    rows, cols = 200, 300
    d = drivers.JacobiSlab(rows, cols, T, drivers.Exchange(), "cuda", fuse=fuse, kernel="wave")
    assert sum(it for it, _ in d.calls()) == T
    opts = dict(backend="agent", order="col")
    assert d.capture(opts)
    assert len(d.graph) == (2 if d.launches_per_step() % 2 else 1)
    d.reset()
    u0 = synth.matrix(4, rows, cols)
    for k in range(1, 4):
        d.step(opts)
        torch.cuda.synchronize()
        assert np.array_equal(d.result().cpu().numpy(), O.jacobi5_f32(u0, k * T)), k


def test_jacobi_driver_world1_graph():
    rows, cols, T = 160, 96, 6
    d = drivers.JacobiSlab(rows, cols, T, drivers.Exchange(), "cuda")
    opts = dict(backend="agent", order="row")
    assert d.capture(opts)
    d.reset()
    d.step(opts)                               # replays the graph
    torch.cuda.synchronize()
    assert np.array_equal(d.result().cpu().numpy(), O.jacobi5_f32(synth.matrix(4, rows, cols), T))


# ---------------------------------------------------------------- G ranks, one GPU
WORKER = textwrap.dedent("""
    import os, sys, numpy as np, torch, torch.distributed as dist
    sys.path.insert(0, {root!r})
    import oracle as O
    from paper_conf_asplos_lis0l0c17_b200 import drivers, shard, synth
    rank, world, cfg = int(sys.argv[1]), int(sys.argv[2]), sys.argv[4]
    dist.init_process_group("gloo", init_method="file://" + sys.argv[3], rank=rank, world_size=world)
    torch.cuda.set_device(0)
    X = drivers.make_exchange("torch", world, rank, 0)
    def rel(got, ref):
        got = np.asarray(got, dtype=np.float64)
        return float(np.max(np.abs(got - ref) / np.abs(ref))) if ref.size else 0.0
    ok, info = True, ""
    if cfg == "atax":
        n, K = 520, 2
        d = drivers.AtaxFamily(n, X, "cuda")
        for _ in range(K):
            d.step(dict(backend="agent", order="col", max_agents=1))
        torch.cuda.synchronize()
        A = synth.matrix(3, n, n)
        x, p, r = synth.uniform(10, n), synth.uniform(11, n), synth.uniform(12, n)
        x1, x2, y1, y2 = synth.uniform(13, n), synth.uniform(14, n), synth.uniform(15, n), synth.uniform(16, n)
        tmp, y = O.atax(A, x)
        q, s = O.bicg(A, p, r)
        o1, o2 = x1, x2
        for _ in range(K):
            o1, o2 = O.mvt(A, np.float32(o1), np.float32(o2), y1, y2)
        lo, hi = d.lo, d.hi
        errs = [rel(d.tmp.cpu(), tmp[lo:hi]), rel(d.q.cpu(), q[lo:hi]), rel(d.x1.cpu(), o1[lo:hi]),
                rel(d.y.cpu(), y), rel(d.s.cpu(), s), rel(d.x2.cpu(), o2)]
        ok, info = max(errs) <= 1e-4, str(errs)
    elif cfg.startswith("jacobi"):
        rows, cols, T = 330, 200, 6
        d = drivers.JacobiSlab(rows, cols, T, X, "cuda", overlap=cfg == "jacobi",
                               halo="fused" if cfg == "jacobi-fused" else "exchange",
                               fuse=int(cfg[-1]) if cfg[:8] in ("jacobi-k", "jacobi-w") else 1,
                               kernel="wave" if cfg.startswith("jacobi-w") else "tile")
        ref = O.jacobi5_f32(synth.matrix(4, rows, cols), T)
        ref2 = O.jacobi5_f32(synth.matrix(4, rows, cols), 2 * T)
        d.step(dict(backend="agent", order="row", max_agents=1))
        torch.cuda.synchronize()
        ok = bool(np.array_equal(d.result().cpu().numpy(), ref[d.lo:d.hi]))
        d.step(dict(backend="agent", order="row", max_agents=1))      # a second step continues the sweeps
        torch.cuda.synchronize()
        ok = ok and bool(np.array_equal(d.result().cpu().numpy(), ref2[d.lo:d.hi]))
        if d.fused:
            ok = ok and int(d.peer.status.item()) == 0
        info = f"overlap={{d.overlap}} fused={{d.fused}}"
    elif cfg.startswith("conv"):
        R = int(cfg[4:])
        rows, cols = 190, 150
        d = drivers.ConvSlab(rows, cols, R, X, "cuda")
        d.step(dict(backend="agent", order="row", max_agents=1))
        torch.cuda.synchronize()
        ref = O.conv2d(synth.matrix(5, rows, cols), d.w)
        got = d.result().cpu().numpy()
        lo, hi = d.lo, d.hi
        inner = ref[lo:hi].copy()
        m = inner != 0
        ok = bool(np.all(got[~m] == 0)) and rel(got[m], inner[m]) <= 1e-4
        info = str(rel(got[m], inner[m]))
    elif cfg.startswith("spmv"):
        d = drivers.SpmvBlock(10, X, "cuda", hot=64 if cfg in ("spmv-hot", "spmv-shub") else 0)
        d.step(dict(backend="agent", order="row", max_agents=1, **({{"shub": True}} if cfg == "spmv-shub" else {{}})))
        torch.cuda.synchronize()
        rp, col = synth.rmat_csr(7, 10, 16)
        val, x = synth.uniform(8, len(col)), synth.uniform(9, len(rp) - 1)
        ref = O.spmv_csr(rp, col, val, x)
        ya = d.yall.cpu().numpy()
        parts = [ya[g * d.cap: g * d.cap + (shard.spmv_row_range(rp, world, g)[1] - shard.spmv_row_range(rp, world, g)[0])]
                 for g in range(world)]
        got = np.concatenate(parts)
        nz = ref != 0
        ok = got.shape == ref.shape and bool(np.all(got[~nz] == 0)) and rel(got[nz], ref[nz]) <= 1e-4
        info = f"rows {{d.lo}}..{{d.hi}}"
    print("RESULT", rank, ok, info, flush=True)
    dist.destroy_process_group()
""")


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return str(p)


@pytest.mark.parametrize("cfg,world", [("atax", 2), ("atax", 4), ("jacobi", 2), ("jacobi", 3), ("jacobi", 4),
                                       ("jacobi-nooverlap", 3), ("jacobi-fused", 2), ("jacobi-fused", 3),
                                       ("jacobi-k4", 2), ("jacobi-k3", 3), ("jacobi-w4", 2), ("jacobi-w5", 3),
                                       ("conv1", 2), ("conv3", 3), ("spmv", 2),
                                       ("spmv", 3), ("spmv-hot", 2), ("spmv-shub", 2)])
def test_sharded_driver_ranks_one_gpu(tmp_path, cfg, world):
    script = tmp_path / "w.py"
    script.write_text(WORKER.format(root=ROOT))
    store = str(tmp_path / "store")            # file rendezvous: no port to race for
    procs = [subprocess.Popen([sys.executable, "-X", "faulthandler", str(script), str(r), str(world), store, cfg],
                              stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True) for r in range(world)]
    outs = []
    for p in procs:
        try:
            outs.append(p.communicate(timeout=300)[0])
        except subprocess.TimeoutExpired:
            p.kill()
            outs.append(p.communicate()[0])
    res = [ln for o in outs for ln in o.splitlines() if ln.startswith("RESULT")]
    if len(res) != world:                       # the whole of every rank's output (faulthandler stacks)
        for r, o in enumerate(outs):
            print(f"---- rank {r} (exit {procs[r].returncode}) ----\n{o}")
    assert len(res) == world, [p.returncode for p in procs]
    assert all(ln.split()[2] == "True" for ln in res), res


@pytest.mark.parametrize("cfg", ["atax", "jacobi", "conv3", "spmv"])
def test_bench_two_ranks_one_gpu(cfg):
    """bench.py's N > 1 path end to end (torchrun, 2 ranks, every rank on GPU 0
    with gloo exchanges -- a harness mode, not a measurement): one JSON line
    from rank 0 with n_gpus 2 and a passing sampled parity probe."""
    import json
    env = dict(os.environ, PYTHONPATH=ROOT)
    size = {"atax": ["--size", "2048"], "jacobi": ["--size", "1024", "--iters", "10"], "conv3": ["--size", "1024"],
            "spmv": ["--size", "14"]}[cfg]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", _port(), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "3", "--warmup", "3", "--config", cfg, "--exchange", "torch",
           "--same-device", "--no-e2e", "--no-cpu-baseline", "--no-graph"] + size
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert out.returncode == 0 and len(lines) == 1, (out.stdout[-3000:], out.stderr[-3000:])
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["parity"]["ok"], d["parity"]


# ---------------------------------------------------------------- fused sweeps (R32)
@pytest.mark.parametrize("fuse", [2, 3, 4])
@pytest.mark.parametrize("v", [dict(backend="agent", order="row"), dict(backend="default"), dict(backend="identity"),
                               dict(backend="static", order="row", num_clusters=148),
                               dict(backend="agent", order="tile", tile=(2, 2))], ids=lambda v: v["backend"])
@pytest.mark.parametrize("rows,cols,T", [(130, 100, 8), (77, 45, 7), (5, 9, 5), (300, 260, 12)])
def test_jacobi_fused_sweeps_bit_exact(fuse, v, rows, cols, T):
    """K sweeps per launch (halo recomputed on chip) equal T single sweeps bit
    for bit, T not a multiple of K included, images smaller than one staged box."""
    u0 = synth.matrix(4, rows, cols)
    a = padded(u0)
    b = padded(np.zeros_like(u0))
    out = ops.jacobi5(a, b, T, fuse=fuse, **v)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), O.jacobi5_f32(u0, T))


def test_jacobi_fused_full_width_sampled():
    """16384 columns (config 3's width), 4 sweeps per launch, 12 sweeps:
    sampled rows and the rows at tile seams, bit-exact."""
    rows, cols, T = 520, 16384, 12
    u0 = synth.matrix(4, rows, cols)
    a = padded(u0)
    out = ops.jacobi5(a, torch.empty_like(a), T, fuse=4, backend="agent", order="row")
    torch.cuda.synchronize()
    ref = O.jacobi5_f32(u0, T)
    got = out.cpu().numpy()
    assert np.array_equal(got[::7], ref[::7])
    assert np.array_equal(got[30:35], ref[30:35]) and np.array_equal(got[255:259], ref[255:259])
