"""GPU parity of CC_K_JACOBI5_WAVE (reading R34): K fused Jacobi sweeps run
by warp agents streaming column strips, carrying every sweep level's last two
rows from one logical CTA to the one below.

Bar: bit-identical to the fp32 oracle (oracle.jacobi5_f32, the single-sweep
PolyBench expression applied `iters` times) for every fuse, backend and
order -- carried and restarted wavefronts alike -- and within 1e-4 of the fp64
oracle; every logical CTA runs exactly once (census), and the map of the
agent / static backends is the plan's partition.
"""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, synth

pytestmark = pytest.mark.gpu
TOL = 1e-4

WVARIANTS = [dict(backend="default"), dict(backend="agent", order="col"), dict(backend="agent", order="row"),
             dict(backend="identity"), dict(backend="agent", order="tile", tile=(2, 3)),
             dict(backend="agent", order="col", batch=1), dict(backend="agent", order="col", batch=7),
             dict(backend="agent", order="col", active_agents=3), dict(backend="agent", order="col", max_agents=5),
             dict(backend="agent", order="col", steal=0, num_clusters=3),
             dict(backend="static", order="col"), dict(backend="static", order="col", num_clusters=5),
             dict(backend="static", order="row", num_clusters=37)]


def dev_padded(u0, ld):
    out = np.zeros((u0.shape[0], ld), np.float32)
    out[:, :u0.shape[1]] = u0
    return torch.from_numpy(out).cuda()


def run(u0, ld, iters, fuse, **v):
    rows, cols = u0.shape
    a = dev_padded(u0, ld).as_strided((rows, cols), (ld, 1))
    b = torch.zeros((rows, ld), device="cuda").as_strided((rows, cols), (ld, 1))
    out = ops.jacobi5_wave(a, b, iters, fuse=fuse, **v)
    torch.cuda.synchronize()
    return out.cpu().numpy()


@pytest.mark.parametrize("v", WVARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("rows,cols,ld,iters,fuse", [(100, 70, 72, 10, 4), (64, 64, 64, 1, 1), (129, 33, 36, 7, 3),
                                                     (5, 3, 4, 3, 2), (300, 250, 252, 9, 4), (261, 241, 244, 13, 8),
                                                     (200, 121, 124, 11, 5), (1, 9, 12, 2, 2), (70, 1, 4, 5, 4),
                                                     (3, 200, 200, 9, 8), (200, 3, 4, 17, 8), (2, 2, 4, 8, 8),
                                                     (65, 113, 116, 16, 8), (64, 112, 112, 0, 8)])
def test_wave_bit_exact(v, rows, cols, ld, iters, fuse):
    u0 = synth.matrix(4, rows, cols)
    got = run(u0, ld, iters, fuse, **v)
    assert np.array_equal(got, O.jacobi5_f32(u0, iters)), v       # same fp32 evaluation order
    assert np.max(np.abs(got - O.jacobi5(u0, iters)) / np.maximum(np.abs(O.jacobi5(u0, iters)), 1e-30)) <= TOL


@pytest.mark.parametrize("fuse", [1, 2, 3, 4, 5, 6, 7, 8])
def test_wave_every_fuse_multi_strip(fuse):
    """Several strips and tile rows, ragged in both directions, iters not a
    multiple of fuse (the tail launch runs fewer sweeps on the same grid)."""
    u0 = synth.matrix(7, 517, 389)
    want = O.jacobi5_f32(u0, 2 * fuse + 1)
    for v in (dict(backend="agent", order="col"), dict(backend="identity"), dict(backend="default")):
        assert np.array_equal(run(u0, 392, 2 * fuse + 1, fuse, **v), want), (fuse, v)


@pytest.mark.parametrize("tile_rows", [8, 16, 100, 256])
@pytest.mark.parametrize("v", [dict(backend="agent", order="col"), dict(backend="default"), dict(backend="identity"),
                               dict(backend="static", order="col", num_clusters=11)],
                         ids=lambda v: "-".join(str(x) for x in v.values()))
def test_wave_tile_rows(v, tile_rows):
    """cc_jacobi5_args.tile_rows: logical CTAs of any height, carried or restarted, bit-exact."""
    u0 = synth.matrix(9, 333, 252)
    a = torch.from_numpy(u0).cuda()
    out = ops.jacobi5_wave(a, torch.zeros_like(a), 19, fuse=8, tile_rows=tile_rows, **v)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), O.jacobi5_f32(u0, 19)), (v, tile_rows)


@pytest.mark.parametrize("v", [dict(backend="agent", order="col"), dict(backend="static", order="col"),
                               dict(backend="identity"), dict(backend="default")],
                         ids=lambda v: "-".join(str(x) for x in v.values()))
def test_wave_census_and_map(v):
    rows, cols = 1000, 700
    u0 = synth.matrix(3, rows, cols)
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    args, flag = cc.jacobi5_args(a, b, 4, fuse=4)
    gx, gy = cc.kernel_grid("jacobi5_wave", args)
    V = gx * gy
    cen = torch.zeros(V, dtype=torch.int32, device="cuda")
    mp = torch.full((V,), -1, dtype=torch.int32, device="cuda")
    kw = dict(v)
    plan = ops.plan_for("jacobi5_wave", args, kw.pop("order", None), None, 0, 0)
    n = cc.launch(plan, "jacobi5_wave", args, cc.make_opts(kw.pop("backend"), census=cen, map=mp, **kw))
    torch.cuda.synchronize()
    assert n == 1
    assert (cen.cpu().numpy() == 1).all()
    if v["backend"] in ("agent", "static"):
        perm, _ = plan.table()
        assert np.array_equal(mp.cpu().numpy(), perm)
    assert np.array_equal((b if flag.value else a).cpu().numpy(), O.jacobi5_f32(u0, 4))


def test_wave_full_size_sampled():
    """Config 3 at full size (16384^2, 100 sweeps, 4 per launch, the bench's
    schedule): sampled cells bit for bit against the fp32 oracle on their
    light cone (radius 100)."""
    N, T = 16384, 100
    u0d = synth.matrix(4, N, N, backend="torch", device="cuda")
    out = ops.jacobi5_wave(u0d, torch.empty_like(u0d), T, fuse=4, backend="agent", order="col")
    torch.cuda.synchronize()
    rng = np.random.default_rng(1)
    pts = [(0, 0), (N - 1, 5), (1, 1), (N // 2, N // 2), (50, N - 2), (64 * 7, 120 * 3), (64 * 7 - 1, 120 * 3 - 1)] + \
          [tuple(rng.integers(0, N, 2)) for _ in range(5)]
    for (i, j) in pts:
        i0, i1 = max(0, i - T), min(N, i + T + 1)
        j0, j1 = max(0, j - T), min(N, j + T + 1)
        win = np.stack([synth.uniform(4, j1 - j0, r * N + j0) for r in range(i0, i1)])
        ref = O.jacobi5_f32(win, T)
        assert out[i, j].item() == ref[i - i0, j - j0], (i, j)


def test_wave_errors():
    a = torch.zeros((64, 64), device="cuda")
    b = torch.zeros_like(a)
    with pytest.raises(cc.CtaclustError):
        ops.jacobi5_wave(a, b, 3, fuse=9)
    with pytest.raises(cc.CtaclustError):
        ops.jacobi5_wave(a, b, 3, fuse=4, backend="tbcluster")
