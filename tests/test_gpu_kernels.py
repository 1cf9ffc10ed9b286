"""GPU parity: every kernel x backend x order against the fp64 CPU oracle.

Bar (BASELINE.json north_star): max relative error <= 1e-4 on positive inputs
(reading R17); integer-valued inputs (reading R18) must match bit for bit; the
Jacobi sweep, which has a fixed fp32 evaluation order, must match the fp32
oracle bit for bit.  Small cases span several tiles and ragged tails; the
full BASELINE sizes are checked on sampled outputs the oracle computes alone.
"""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, synth

pytestmark = pytest.mark.gpu
TOL = 1e-4

VARIANTS = [
    dict(backend="default"),
    dict(backend="agent", order="row"),
    dict(backend="agent", order="col"),
    dict(backend="agent", order="tile", tile=(4, 4)),
    dict(backend="agent", order="col", active_agents=1),
    dict(backend="agent", order="col", stages=1),
    dict(backend="agent", order="col", stages=6, batch=3),
    dict(backend="identity"),
    dict(backend="redirect", order="row"),
    dict(backend="default", staging="direct"),
    dict(backend="agent", order="col", staging="direct"),
    dict(backend="agent", order="row", staging="tma", stages=3, batch=2),
    dict(backend="agent", order="col", l2_hint="both"),
    dict(backend="agent", order="col", staging="direct", l2_hint="both", carveout=50),
    dict(backend="identity", l2_hint="stream_first", carveout=0),
    dict(backend="default", carveout=100),
    dict(backend="static", order="col"),
    dict(backend="static", order="row", num_clusters=592, stages=3),
    dict(backend="static", order="tile", tile=(2, 2), num_clusters=5, staging="direct"),
]


def relerr(got, ref):
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    den = np.maximum(np.abs(ref), 1e-30)
    return float(np.max(np.abs(got - ref) / den)) if ref.size else 0.0


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def padded(A, ld):
    out = np.zeros((A.shape[0], ld), np.float32)
    out[:, :A.shape[1]] = A
    return dev(out)


def mat(seed, m, n, kind="uniform"):
    return synth.matrix(seed, m, n, kind=kind)


# ---------------------------------------------------------------- matvec
@pytest.mark.parametrize("v", VARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("m,n,ld", [(1024, 1024, 1024), (1000, 1001, 1004), (33, 7, 8)])
def test_matvec(v, m, n, ld):
    A = mat(1, m, n)
    x = synth.uniform(2, n)
    Ad = padded(A, ld).as_strided((m, n), (ld, 1))
    y = ops.matvec(Ad, dev(x), **v)
    torch.cuda.synchronize()
    assert relerr(y.cpu().numpy(), O.matvec(A, x)) <= TOL


@pytest.mark.parametrize("v", VARIANTS[:4], ids=lambda v: "-".join(str(x) for x in v.values()))
def test_matvec_integer_exact(v):
    A = mat(3, 300, 200, "int")
    x = synth.small_int(4, 200)
    y = ops.matvec(dev(A), dev(x), **v)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().astype(np.float64), O.matvec(A, x))


# ---------------------------------------------------------------- ATAX / BICG / MVT
def _family(A, Ad, m, n, v, seed=10):
    x = synth.uniform(seed, n); p = synth.uniform(seed + 1, n); r = synth.uniform(seed + 2, m)
    x1 = synth.uniform(seed + 3, m); x2 = synth.uniform(seed + 4, n)
    y1 = synth.uniform(seed + 5, n); y2 = synth.uniform(seed + 6, m)
    tmp, y = ops.atax(Ad, dev(x), **v)
    q, s = ops.bicg(Ad, dev(p), dev(r), **v)
    X1, X2 = dev(x1), dev(x2)
    ops.mvt(Ad, dev(y1), dev(y2), X1, X2, **v)
    torch.cuda.synchronize()
    return (x, p, r, x1, x2, y1, y2), (tmp.cpu().numpy(), y.cpu().numpy(), q.cpu().numpy(),
                                      s.cpu().numpy(), X1.cpu().numpy(), X2.cpu().numpy())


@pytest.mark.parametrize("v", VARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("m,n,ld", [(1000, 1001, 1004), (2048, 4096, 4096), (31, 257, 260)])
def test_atax_bicg_mvt(v, m, n, ld):
    A = mat(9, m, n)
    Ad = padded(A, ld).as_strided((m, n), (ld, 1))
    (x, p, r, x1, x2, y1, y2), (tmp, y, q, s, X1, X2) = _family(A, Ad, m, n, v)
    rt, ry = O.atax(A, x)
    assert relerr(tmp, rt) <= TOL
    assert relerr(y, O.atax_pass2(A, tmp)) <= TOL          # pass 2 on the GPU's own fp32 tmp
    assert relerr(y, ry) <= TOL
    rq, rs = O.bicg(A, p, r)
    assert relerr(q, rq) <= TOL and relerr(s, rs) <= TOL
    r1, r2 = O.mvt(A, x1, x2, y1, y2)
    assert relerr(X1, r1) <= TOL and relerr(X2, r2) <= TOL


@pytest.mark.parametrize("v", VARIANTS[:3] + VARIANTS[6:], ids=lambda v: "-".join(str(x) for x in v.values()))
def test_bicg_integer_exact(v):
    m, n = 700, 900
    A = mat(11, m, n, "int")
    p, r = synth.small_int(12, n), synth.small_int(13, m)
    q, s = ops.bicg(dev(A), dev(p), dev(r), **v)
    torch.cuda.synchronize()
    rq, rs = O.bicg(A, p, r)
    assert np.array_equal(q.cpu().numpy().astype(np.float64), rq)
    assert np.array_equal(s.cpu().numpy().astype(np.float64), rs)


def test_bicg_full_size_config2():
    """BASELINE config 2 at full size n = 16384 (the bench's launch config:
    agent backend, column clustering), every output checked."""
    n = 16384
    A = synth.matrix(3, n, n)                      # 1 GiB, host, from the shared generator
    p, r = synth.uniform(31, n), synth.uniform(32, n)
    q, s = ops.bicg(dev(A), dev(p), dev(r), backend="agent", order="col")
    torch.cuda.synchronize()
    rq, rs = O.bicg(A, p, r)
    assert relerr(q.cpu().numpy(), rq) <= TOL and relerr(s.cpu().numpy(), rs) <= TOL


def test_atax_mvt_full_size_config2():
    """BASELINE config 2 at full size n = 16384 for the other two kernels of the
    bench step (ATAX two passes, MVT fused), in the bench's launch config
    (agent backend, column clustering) and the static binding: every output."""
    n = 16384
    A = synth.matrix(3, n, n)
    Ad = dev(A)
    x, y1, y2 = synth.uniform(10, n), synth.uniform(15, n), synth.uniform(16, n)
    x1, x2 = synth.uniform(13, n), synth.uniform(14, n)
    rtmp, ry = O.atax(A, x)
    r1, r2 = O.mvt(A, x1, x2, y1, y2)
    for v in (dict(backend="agent", order="col"), dict(backend="static", order="col", num_clusters=444)):
        tmp, y = ops.atax(Ad, dev(x), **v)
        X1, X2 = dev(x1), dev(x2)
        ops.mvt(Ad, dev(y1), dev(y2), X1, X2, **v)
        torch.cuda.synchronize()
        assert relerr(tmp.cpu().numpy(), rtmp) <= TOL and relerr(y.cpu().numpy(), ry) <= TOL, v
        assert relerr(X1.cpu().numpy(), r1) <= TOL and relerr(X2.cpu().numpy(), r2) <= TOL, v


FUSED_VARIANTS = [dict(backend="agent"), dict(backend="identity"), dict(backend="static", num_clusters=148),
                  dict(backend="static", num_clusters=444), dict(backend="agent", active_agents=1, stages=2),
                  dict(backend="agent", steal=0), dict(backend="default")]


@pytest.mark.parametrize("v", FUSED_VARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("m,n,ld", [(1000, 1001, 1004), (300, 16384, 16384), (7, 13, 16), (1, 1, 4), (150, 4096, 4100)])
def test_atax_fused(v, m, n, ld):
    """One-pass ATAX (CC_K_ATAX_FUSED): tmp and y vs the oracle; y also vs
    pass 2 on the GPU's own fp32 tmp; ragged n (padding in the staged row must
    not leak), m below and above the SM count, n at the 16384 limit."""
    A = mat(9, m, n)
    Ad = padded(A, ld).as_strided((m, n), (ld, 1))
    if ld > n:                                             # poison the padding: it must be ignored
        Ad.as_strided((m, ld), (ld, 1))[:, n:] = float("nan")
    x = synth.uniform(10, n)
    tmp, y = ops.atax_fused(Ad, dev(x), **v)
    torch.cuda.synchronize()
    rt, ry = O.atax(A, x)
    assert relerr(tmp.cpu().numpy(), rt) <= TOL
    assert relerr(y.cpu().numpy(), O.atax_pass2(A, tmp.cpu().numpy())) <= TOL
    assert relerr(y.cpu().numpy(), ry) <= TOL


def test_atax_fused_integer_exact_and_census():
    m, n = 200, 98                      # every partial sum of tmp and y stays below 2^24
    A = mat(11, m, n, "int")
    Ad = padded(A, 100).as_strided((m, n), (100, 1))
    x = synth.small_int(12, n)
    cen = torch.zeros(m, dtype=torch.int32, device="cuda")
    tmp, y = ops.atax_fused(Ad, dev(x), backend="agent", census=cen)
    torch.cuda.synchronize()
    rt, ry = O.atax(A, x)
    assert np.array_equal(tmp.cpu().numpy().astype(np.float64), rt)
    assert np.array_equal(y.cpu().numpy().astype(np.float64), ry)
    assert bool(torch.all(cen == 1))


def test_atax_fused_full_size_config2():
    """Config 2's ATAX at n = 16384 in the bench's launch config (agent, one
    row per logical CTA), every output."""
    n = 16384
    A = synth.matrix(3, n, n)
    x = synth.uniform(10, n)
    tmp, y = ops.atax_fused(dev(A), dev(x), backend="agent")
    torch.cuda.synchronize()
    rt, ry = O.atax(A, x)
    assert relerr(tmp.cpu().numpy(), rt) <= TOL and relerr(y.cpu().numpy(), ry) <= TOL


def test_atax_fused_limits():
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    with pytest.raises(cc.CtaclustError) as e:
        ops.atax_fused(torch.zeros(4, 16388, device="cuda"), torch.zeros(16388, device="cuda"))
    assert e.value.status == -6


def test_matvec_config1_static_binding():
    """Config 1 (n = 1024, 32 x 32 tiles) in the configuration that measures
    fastest (static binding, M = 3 x SMs, row clustering) and the agent."""
    A, x = mat(1, 1024, 1024), synth.uniform(2, 1024)
    ref = O.matvec(A, x)
    for v in (dict(backend="static", order="row", num_clusters=444), dict(backend="static", order="row", num_clusters=296),
              dict(backend="agent", order="row")):
        y = ops.matvec(dev(A), dev(x), **v)
        torch.cuda.synchronize()
        assert relerr(y.cpu().numpy(), ref) <= TOL, v


# ---------------------------------------------------------------- Jacobi
JVARIANTS = [dict(backend="default"), dict(backend="agent", order="tile", tile=(8, 8)),
             dict(backend="agent", order="row"), dict(backend="agent", order="col", active_agents=2),
             dict(backend="agent", order="tile", tile=(2, 2), stages=8, batch=7), dict(backend="identity"),
             dict(backend="redirect", order="tile", tile=(4, 4)),
             dict(backend="default", staging="l1"), dict(backend="default", staging="direct"),
             dict(backend="agent", order="tile", tile=(8, 8), staging="l1"),
             dict(backend="agent", order="row", staging="direct"),
             dict(backend="agent", order="row", l2_hint="both"),
             dict(backend="agent", order="row", staging="l1", l2_hint="both", carveout=25),
             dict(backend="static", order="row", num_clusters=592), dict(backend="static", order="tile", tile=(2, 2)),
             dict(backend="agent", order="row", l2_hint="halo_last"),
             dict(backend="static", order="row", num_clusters=296, l2_hint="halo_last_stream_first")]


@pytest.mark.parametrize("v", JVARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("rows,cols,ld,iters", [(100, 70, 72, 10), (64, 64, 64, 1), (129, 33, 36, 7), (5, 3, 4, 3)])
def test_jacobi_bit_exact(v, rows, cols, ld, iters):
    u0 = mat(4, rows, cols)
    a, b = padded(u0, ld), torch.zeros((rows, ld), device="cuda")
    a = a.as_strided((rows, cols), (ld, 1)); b = b.as_strided((rows, cols), (ld, 1))
    out = ops.jacobi5(a, b, iters, **v)
    torch.cuda.synchronize()
    got = out.cpu().numpy()
    assert np.array_equal(got, O.jacobi5_f32(u0, iters))      # same fp32 evaluation order
    assert relerr(got, O.jacobi5(u0, iters)) <= TOL


def test_jacobi_full_size_sampled():
    """Config 3 at full size (16384^2, 100 sweeps): sampled cells checked bit for
    bit against the fp32 oracle run on the light cone (radius = iters) around
    each sample; outside the cone nothing can reach the sample in 100 sweeps."""
    N, T = 16384, 100
    u0d = synth.matrix(4, N, N, backend="torch", device="cuda")
    out = ops.jacobi5(u0d, torch.empty_like(u0d), T, backend="agent", order="tile", tile=(8, 8))
    torch.cuda.synchronize()
    rng = np.random.default_rng(0)
    pts = [(0, 0), (N - 1, 5), (1, 1), (N // 2, N // 2), (50, N - 2)] + \
          [tuple(rng.integers(0, N, 2)) for _ in range(6)]
    for (i, j) in pts:
        i0, i1 = max(0, i - T), min(N, i + T + 1)
        j0, j1 = max(0, j - T), min(N, j + T + 1)
        win = np.stack([synth.uniform(4, j1 - j0, r * N + j0) for r in range(i0, i1)])
        ref = O.jacobi5_f32(win, T)
        # cells of the window edge that are not true boundary are "fixed" in the
        # oracle run; the sample sits >= T cells away from any such edge.
        assert out[i, j].item() == ref[i - i0, j - j0], (i, j)


# ---------------------------------------------------------------- conv2d
CVARIANTS = [dict(backend="default"), dict(backend="agent", order="tile", tile=(8, 8)),
             dict(backend="agent", order="col", stages=1, batch=1), dict(backend="identity"),
             dict(backend="tbcluster", cluster_size=1), dict(backend="tbcluster", cluster_size=2),
             dict(backend="tbcluster", cluster_size=4), dict(backend="tbcluster", cluster_size=8),
             dict(backend="redirect", order="row"),
             dict(backend="default", staging="l1"), dict(backend="default", staging="direct"),
             dict(backend="agent", order="tile", tile=(8, 8), staging="l1"),
             dict(backend="agent", order="col", staging="direct"),
             dict(backend="agent", order="row", l2_hint="both", carveout=100),
             dict(backend="static", order="row", num_clusters=740), dict(backend="static", order="col", staging="direct"),
             dict(backend="agent", order="row", l2_hint="halo_last"),
             dict(backend="agent", order="tile", tile=(4, 4), l2_hint="halo_last_stream_first"),
             dict(backend="static", order="row", num_clusters=296, l2_hint="halo_last")]


@pytest.mark.parametrize("v", CVARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("R", [1, 3])
@pytest.mark.parametrize("rows,cols,ld", [(100, 70, 72), (300, 257, 260), (7, 9, 12)])
def test_conv2d(v, R, rows, cols, ld):
    img = mat(5, rows, cols)
    w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
    w = w / w.sum()
    a = padded(img, ld).as_strided((rows, cols), (ld, 1))
    o = torch.full((rows, ld), 7.0, device="cuda").as_strided((rows, cols), (ld, 1))
    ops.conv2d(a, w, out=o, **v)
    torch.cuda.synchronize()
    ref = O.conv2d(img, w)
    got = o.cpu().numpy()
    assert np.all(got[ref == 0] == 0)
    nz = ref != 0
    assert relerr(got[nz], ref[nz]) <= TOL


@pytest.mark.parametrize("v", CVARIANTS[:2] + CVARIANTS[5:6], ids=lambda v: "-".join(str(x) for x in v.values()))
def test_conv2d_integer_exact_signed(v):
    """Signed PolyBench 2DCONV 3x3 constants are not integers; use an integer
    signed filter so the exact-mode comparison is bit-for-bit (reading R18)."""
    img = mat(7, 200, 152, "int")
    w = np.array([[1, -2, 3], [-4, 5, -6], [7, -8, 2]], np.float32)
    o = ops.conv2d(dev(img), w, **v)
    torch.cuda.synchronize()
    assert np.array_equal(o.cpu().numpy().astype(np.float64), O.conv2d(img, w))


def test_conv2d_full_size_sampled():
    N = 8192
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    for R in (1, 3):
        w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
        w = w / w.sum()
        for v in (dict(backend="agent", order="tile", tile=(8, 8)), dict(backend="tbcluster", cluster_size=4)):
            o = ops.conv2d(img, w, **v)
            torch.cuda.synchronize()
            rng = np.random.default_rng(R)
            for (i, j) in [(R, R), (N - 1 - R, N - 1 - R), (0, 5)] + [tuple(rng.integers(0, N, 2)) for _ in range(20)]:
                i0, i1, j0, j1 = max(0, i - R), min(N, i + R + 1), max(0, j - R), min(N, j + R + 1)
                win = np.stack([synth.uniform(5, j1 - j0, r * N + j0) for r in range(i0, i1)])
                if R <= i < N - R and R <= j < N - R:
                    ref = float(O.conv2d(win, w)[R, R])      # the oracle on the (2R+1)^2 window
                    assert abs(o[i, j].item() - ref) <= TOL * abs(ref), (R, i, j, v)
                else:
                    assert o[i, j].item() == 0.0


def _user_orders(gx, gy):
    """USER-order plans (reading of the paper's user-defined partition): a
    random permutation and the time-aligned interleaved row order."""
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    M = cc.device_info(0)["num_sms"]
    V, c = gx * gy, 2
    K = (V + c - 1) // c
    ilv = np.concatenate([np.arange(k * c, min(V, (k + 1) * c)) for i in range(M) for k in range(i, K, M)])
    rnd = np.random.default_rng(gx * 131 + gy).permutation(V)
    return [("ilv", ilv.astype(np.int32)), ("rand", rnd.astype(np.int32))]


@pytest.mark.parametrize("backend", ["agent", "static"])
@pytest.mark.parametrize("rows,cols,ld", [(300, 257, 260), (100, 70, 72)])
def test_stencils_user_order(backend, rows, cols, ld):
    """Jacobi (bit-exact vs the fp32 oracle) and conv 3x3 / 7x7 under USER orders."""
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    u0 = mat(4, rows, cols)
    a = padded(u0, ld).as_strided((rows, cols), (ld, 1))
    b = torch.zeros((rows, ld), device="cuda").as_strided((rows, cols), (ld, 1))
    args, _ = cc.jacobi5_args(a, b, 1)
    gx, gy = cc.kernel_grid("jacobi5", args)
    ref_j = O.jacobi5_f32(u0, 5)
    for name, uo in _user_orders(gx, gy):
        a.copy_(torch.from_numpy(u0).cuda())
        out = ops.jacobi5(a, b, 5, backend=backend, user_order=uo, num_clusters=0 if backend == "agent" else 296)
        torch.cuda.synchronize()
        assert np.array_equal(out.cpu().numpy(), ref_j), name
    img = mat(5, rows, cols)
    a.copy_(torch.from_numpy(img).cuda())
    for R in (1, 3):
        w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
        w = w / w.sum()
        ref = O.conv2d(img, w)
        args, _w = cc.conv2d_args(a, b, w)
        gx, gy = cc.kernel_grid("conv2d", args)
        for name, uo in _user_orders(gx, gy):
            b.fill_(7.0)
            ops.conv2d(a, w, out=b, backend=backend, user_order=uo, num_clusters=0 if backend == "agent" else 296)
            torch.cuda.synchronize()
            got = b.cpu().numpy()
            assert np.all(got[ref == 0] == 0), (R, name)
            nz = ref != 0
            assert relerr(got[nz], ref[nz]) <= TOL, (R, name)


# ---------------------------------------------------------------- SpMV
def _csr_dev(rp, col, val):
    return ops.SpmvMatrix(dev(rp.astype(np.int32)), dev(col.astype(np.int32)), dev(val.astype(np.float32)))


SVARIANTS = [dict(backend="default"), dict(backend="agent", order="row"), dict(backend="agent", active_agents=1),
             dict(backend="agent", stages=4, batch=5), dict(backend="identity"), dict(backend="redirect"),
             dict(backend="agent", order="row", l2_hint="both"), dict(backend="default", carveout=0),
             dict(backend="static", order="row", num_clusters=740), dict(backend="static", order="row", num_clusters=3)]


def _edge_matrices():
    # empty rows, a giant row spanning many logical CTAs, tiny rows
    n = 5000
    deg = np.zeros(n, np.int64)
    deg[7] = 20000 % n + 3000
    deg[100:4000:3] = 1
    deg[4500] = 4999
    deg[-1] = 2
    rp = np.zeros(n + 1, np.int64); np.cumsum(deg, out=rp[1:])
    col = np.concatenate([np.sort(synth.random_permutation(int(i), n)[:d]) for i, d in enumerate(deg) if d])
    yield "edges", rp, col, n
    rp2 = np.zeros(301, np.int64)
    yield "all-empty", rp2, np.zeros(0, np.int64), 300
    rp3, col3 = synth.rmat_csr(7, 12, 16)
    yield "rmat12", rp3.astype(np.int64), col3, 1 << 12
    # mostly-empty rows: every logical CTA spans > SPMV_ROWCAP rows, so the
    # merge walk reads its row ends from global memory (k_spmv.cuh)
    n4 = 100003
    deg4 = np.zeros(n4, np.int64)
    deg4[::37] = 2
    rp4 = np.zeros(n4 + 1, np.int64); np.cumsum(deg4, out=rp4[1:])
    k4 = int(deg4.sum()) // 2
    c0 = (synth.uniform(12, k4) * (n4 - 1)).astype(np.int64)
    c1 = (c0 + 1 + (synth.uniform(13, k4) * (n4 - 2)).astype(np.int64)) % n4   # != c0
    col4 = np.sort(np.stack([c0, c1], 1), axis=1).reshape(-1)
    yield "mostly-empty", rp4, col4, n4


@pytest.mark.parametrize("v", SVARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
def test_spmv(v):
    for name, rp, col, n in _edge_matrices():
        val = synth.uniform(8, len(col))
        x = synth.uniform(9, n)
        Am = _csr_dev(rp, col, val)
        y = ops.spmv(Am, dev(x), **v)
        torch.cuda.synchronize()
        ref = O.spmv_csr(rp.astype(np.int32), col.astype(np.int32), val, x)
        got = y.cpu().numpy()
        nz = ref != 0
        assert np.all(got[~nz] == 0), name
        assert relerr(got[nz], ref[nz]) <= TOL, name
        # integer-exact mode
        vi, xi = synth.small_int(10, len(col)), synth.small_int(11, n)
        Am = _csr_dev(rp, col, vi)
        y = ops.spmv(Am, dev(xi), **v)
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy().astype(np.float64),
                              O.spmv_csr(rp.astype(np.int32), col.astype(np.int32), vi, xi)), name


@pytest.mark.parametrize("hot", [1, 64, 100000])
def test_spmv_hub_form(hot):
    """Hub-column form (cc_spmv_inspect, P:1925 inspector): the inspector picks
    the most-referenced columns (every hub's degree >= every other column's),
    the encoding decodes back to col, and y has the plain form's bits under
    every backend (same products, same order) and matches the oracle."""
    for name, rp, col, n in _edge_matrices():
        val = synth.uniform(8, len(col))
        x = synth.uniform(9, n)
        plain = _csr_dev(rp, col, val)
        Am = ops.SpmvMatrix(plain.row_ptr, plain.col, plain.val, hot=hot)
        deg = np.bincount(col, minlength=n) if len(col) else np.zeros(n, np.int64)
        hubs = Am.hot[: Am.n_hot].cpu().numpy()
        assert Am.n_hot == min(hot, int(np.count_nonzero(deg))), name
        assert len(set(hubs.tolist())) == Am.n_hot
        if Am.n_hot:
            rest = np.setdiff1d(np.arange(n), hubs)
            assert deg[hubs].min() >= (deg[rest].max() if rest.size else 0), name
            dh = np.minimum(deg[hubs], 65535)
            T = min(Am.n_hot, cc.SPMV_SHUB_SLOTS)               # the shared-memory tier: the hottest slots
            assert T == Am.n_hot or dh[:T].min() >= dh[T:].max(), name
        enc = Am.col_kernel.cpu().numpy()
        dec = enc.copy()
        neg = enc < 0
        dec[neg] = hubs[-enc[neg] - 1]
        assert np.array_equal(dec, col), name
        ref = O.spmv_csr(rp.astype(np.int32), col.astype(np.int32), val, x)
        for v in (dict(backend="default"), dict(backend="agent", order="row"), dict(backend="identity"),
                  dict(backend="static", order="row", num_clusters=740), dict(backend="agent", l2_hint="both")):
            y0 = ops.spmv(plain, dev(x), **v)
            y1 = ops.spmv(Am, dev(x), **v)
            torch.cuda.synchronize()
            got = y1.cpu().numpy()
            nz = ref != 0
            assert np.all(got[~nz] == 0), (name, v)
            assert relerr(got[nz], ref[nz]) <= TOL, (name, v)
            if v["backend"] in ("default", "static"):     # deterministic schedules: the same bits
                assert np.array_equal(got, y0.cpu().numpy()), (name, v)


SHUB_VARIANTS = [dict(backend="agent", order="row"), dict(backend="identity"),
                 dict(backend="static", order="row", num_clusters=740), dict(backend="static", order="row", num_clusters=3),
                 dict(backend="agent", order="row", stages=6, batch=5), dict(backend="agent", order="row", steal=0),
                 dict(backend="agent", order="row", l2_hint="both"), dict(backend="agent", order="col")]


@pytest.mark.parametrize("hot", [0, 1, 7, 64, 43008])
def test_spmv_shub(hot):
    """CC_K_SPMV_SHUB (hub array in each agent's shared memory, one bulk copy
    per agent): the oracle's y under every persistent schedule, including the
    hub tail that is not a multiple of 16 bytes (n_hot = 1, 7), an all-hub
    matrix (rmat12: every column a hub slot) and plain CSR (hot = 0); bit-exact
    in the integer-exact mode."""
    for name, rp, col, n in _edge_matrices():
        val = synth.uniform(8, len(col))
        x = synth.uniform(9, n)
        plain = _csr_dev(rp, col, val)
        Am = ops.SpmvMatrix(plain.row_ptr, plain.col, plain.val, hot=hot) if hot else plain
        ref = O.spmv_csr(rp.astype(np.int32), col.astype(np.int32), val, x)
        vi, xi = synth.small_int(10, len(col)), synth.small_int(11, n)
        Ai = ops.SpmvMatrix(plain.row_ptr, plain.col, dev(vi.astype(np.float32)), hot=hot) if hot else \
            _csr_dev(rp, col, vi)
        refi = O.spmv_csr(rp.astype(np.int32), col.astype(np.int32), vi, xi)
        for v in SHUB_VARIANTS:
            y = ops.spmv(Am, dev(x), shub=True, **v)
            torch.cuda.synchronize()
            got = y.cpu().numpy()
            nz = ref != 0
            assert np.all(got[~nz] == 0), (name, v)
            assert relerr(got[nz], ref[nz]) <= TOL, (name, v)
            yi = ops.spmv(Ai, dev(xi), shub=True, **v)
            torch.cuda.synchronize()
            assert np.array_equal(yi.cpu().numpy().astype(np.float64), refi), (name, v)


def test_spmv_shub_tiers():
    """SHUB is for persistent agents only; with more hub slots than its
    shared-memory tier (include/ctaclust.h CC_SPMV_SHUB_SLOTS) the colder
    slots are read from the L1 array -- both tiers against the oracle, and
    bit-exact in the integer-exact mode."""
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    rp, col = synth.rmat_csr(7, 17, 16)
    n = len(rp) - 1
    val, x = synth.uniform(8, len(col)), synth.uniform(9, n)
    plain = _csr_dev(rp, col, val)
    for b in ("default", "redirect"):
        with pytest.raises(cc.CtaclustError):
            ops.spmv(plain, dev(x), backend=b, shub=True)
    ref = O.spmv_csr(rp.astype(np.int32), col.astype(np.int32), val, x)
    vi, xi = synth.small_int(10, len(col)), synth.small_int(11, n)
    refi = O.spmv_csr(rp.astype(np.int32), col.astype(np.int32), vi, xi)
    for hot in (cc.SPMV_SHUB_SLOTS - 1, cc.SPMV_SHUB_SLOTS + 3, cc.SPMV_SHUB_SLOTS + 6, 3 * cc.SPMV_SHUB_SLOTS):
        Am = ops.SpmvMatrix(plain.row_ptr, plain.col, plain.val, hot=hot)
        Ai = ops.SpmvMatrix(plain.row_ptr, plain.col, dev(vi.astype(np.float32)), hot=hot)
        assert Am.n_hot == hot
        for v in (dict(backend="agent", order="row"), dict(backend="identity"),
                  dict(backend="static", order="row", num_clusters=296)):
            y = ops.spmv(Am, dev(x), shub=True, **v)
            yi = ops.spmv(Ai, dev(xi), shub=True, **v)
            torch.cuda.synchronize()
            nz = ref != 0
            assert relerr(y.cpu().numpy()[nz], ref[nz]) <= TOL, (hot, v)
            assert np.array_equal(yi.cpu().numpy().astype(np.float64), refi), (hot, v)


def test_spmv_full_size_sampled():
    """Config 5 at full size (R-MAT scale 24, edge factor 16, ~263 M nnz) in the
    bench suite's launch configs: 3000 sampled rows plus the 20 heaviest rows
    (the power-law hubs, spanning many logical CTAs) checked against the oracle
    run on exactly those rows."""
    rp, col = synth.rmat_csr(7, 24, 16, backend="torch", device="cuda")
    nnz, n = col.numel(), rp.numel() - 1
    val = synth.uniform(8, nnz, backend="torch", device="cuda")
    x = synth.uniform(9, n, backend="torch", device="cuda")
    Am = ops.SpmvMatrix(rp, col, val)
    rph = rp.cpu().numpy().astype(np.int64)
    deg = np.diff(rph)
    rng = np.random.default_rng(5)
    rows = np.unique(np.concatenate([rng.integers(0, n, 3000), np.argsort(deg)[-20:], [0, n - 1]]))
    sub_rp = np.zeros(rows.size + 1, np.int64)
    np.cumsum(deg[rows], out=sub_rp[1:])
    idx = torch.from_numpy(np.concatenate([np.arange(rph[r], rph[r + 1]) for r in rows])).cuda()
    sub_col = col[idx].cpu().numpy()
    sub_val = val[idx].cpu().numpy()
    ref = O.spmv_csr(sub_rp.astype(np.int32), sub_col.astype(np.int32), sub_val, x.cpu().numpy())
    Ah = ops.SpmvMatrix(rp, col, val, hot=16384)
    As = ops.SpmvMatrix(rp, col, val, hot=43008)
    for M, v in ((Am, dict(backend="default")), (Am, dict(backend="agent", order="row")),
                 (Am, dict(backend="identity")), (Ah, dict(backend="agent", order="row")),
                 (Ah, dict(backend="default")), (As, dict(backend="agent", order="row", shub=True)),
                 (As, dict(backend="identity", shub=True))):
        y = ops.spmv(M, x, **v)
        torch.cuda.synchronize()
        got = y[torch.from_numpy(rows).cuda()].cpu().numpy()
        nz = ref != 0
        assert np.all(got[~nz] == 0), v
        assert relerr(got[nz], ref[nz]) <= TOL, v


# ---- S8(f)3: 64-bin histogram (HST, reading R24) -- integer counts, bit-exact ----
HVARIANTS = [dict(backend="default"), dict(backend="agent", order="row"), dict(backend="agent", order="col"),
             dict(backend="identity"), dict(backend="redirect", order="row"),
             dict(backend="default", staging="direct"), dict(backend="agent", order="row", staging="direct"),
             dict(backend="agent", order="row", staging="l1"), dict(backend="agent", order="row", active_agents=1),
             dict(backend="agent", order="row", stages=4, batch=3), dict(backend="agent", order="row", stages=1),
             dict(backend="agent", order="row", l2_hint="both"), dict(backend="static", order="row", num_clusters=888),
             dict(backend="static", order="row", num_clusters=2, staging="direct")]


@pytest.mark.parametrize("v", HVARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
def test_hist64(v):
    for n in (0, 1, 15, 16, 17, 32768, 32769, 100003, 5 * 32768 + 7):
        for kind in ("uniform", "skewed"):
            data = synth.bytes_u8(30 + n % 7, n, kind=kind)
            got = ops.hist64(torch.from_numpy(data).cuda(), **v)
            torch.cuda.synchronize()
            ref = O.hist64(data)
            assert np.array_equal(got.cpu().numpy().view(np.uint32).astype(np.uint64), ref), (n, kind)


def test_hist64_full_size_and_errors():
    n = 1 << 30
    data = synth.bytes_u8(31, n, backend="torch", device="cuda")
    ref = O.hist64(data.cpu().numpy())
    for v in (dict(backend="default"), dict(backend="agent", order="row")):
        got = ops.hist64(data, **v)
        torch.cuda.synchronize()
        assert np.array_equal(got.cpu().numpy().view(np.uint32).astype(np.uint64), ref), v
    with pytest.raises(Exception):
        ops.hist64(data[1:1025])                  # not 16-byte aligned


# ---------------------------------------------------------------- degenerate sizes
DEG_BACKENDS = [dict(backend="default"), dict(backend="agent", order="row"), dict(backend="agent", order="col"),
                dict(backend="static", order="row"), dict(backend="identity")]


@pytest.mark.parametrize("v", DEG_BACKENDS, ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("m,n", [(0, 5), (5, 0), (1, 1), (1, 4), (3, 1), (0, 0)])
def test_gemv_family_degenerate(v, m, n):
    """Empty and one-element operands: y = A x over an empty dimension is the
    zero vector (an empty sum), never uninitialised memory."""
    ld = max(4, (n + 3) // 4 * 4)
    A = mat(3, m, n)
    Ad = padded(A, ld).as_strided((m, n), (ld, 1)) if m > 0 else torch.zeros((0, ld), device="cuda")[:, :n]
    x, p, r = synth.uniform(10, n), synth.uniform(11, n), synth.uniform(12, m)
    yz = ops.matvec(Ad, dev(x), **v)                              # zero-initialised y
    q, s = ops.bicg(Ad, dev(p), dev(r), **v)
    tmp, yy = ops.atax(Ad, dev(x), **v)
    torch.cuda.synchronize()
    np.testing.assert_allclose(yz.cpu().numpy(), O.matvec(A, x), rtol=TOL, atol=0)
    rq, rs = O.bicg(A, p, r)
    np.testing.assert_allclose(q.cpu().numpy(), rq, rtol=TOL, atol=0)
    np.testing.assert_allclose(s.cpu().numpy(), rs, rtol=TOL, atol=0)
    rt, ry = O.atax(A, x)
    np.testing.assert_allclose(tmp.cpu().numpy(), rt, rtol=TOL, atol=0)
    np.testing.assert_allclose(yy.cpu().numpy(), ry, rtol=TOL, atol=0)


@pytest.mark.parametrize("v", DEG_BACKENDS + [dict(backend="tbcluster", cluster_size=2)],
                         ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("rows,cols", [(1, 1), (2, 2), (3, 3), (5, 5), (1, 40), (40, 1)])
def test_stencils_degenerate(v, rows, cols):
    """Grids with no interior (Jacobi keeps the boundary; conv outputs are all
    border zeros when the image is smaller than the filter) and one-cell-wide
    interiors."""
    ld = max(4, (cols + 3) // 4 * 4)
    img = mat(5, rows, cols)
    a = padded(img, ld).as_strided((rows, cols), (ld, 1))
    for R in (1, 3):
        w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
        o = torch.full((rows, ld), 7.0, device="cuda").as_strided((rows, cols), (ld, 1))
        ops.conv2d(a, w, out=o, **v)
        torch.cuda.synchronize()
        ref = O.conv2d(img, w)
        got = o.cpu().numpy()
        assert np.all(got[ref == 0] == 0), (R, v)
        nz = ref != 0
        assert relerr(got[nz], ref[nz]) <= TOL, (R, v)
    if v["backend"] == "tbcluster":
        return
    b = torch.full((rows, ld), 7.0, device="cuda").as_strided((rows, cols), (ld, 1))
    a2 = padded(img, ld).as_strided((rows, cols), (ld, 1))
    out = ops.jacobi5(a2, b, 3, **v)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), O.jacobi5_f32(img, 3)), v


def test_spmv_with_l2_persisting_x():
    """cc_l2_persist: results unchanged with x held L2-persisting on the stream,
    and the window clears."""
    from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc
    rp, col = synth.rmat_csr(7, 12, 16)
    val, x = synth.uniform(8, len(col)), synth.uniform(9, len(rp) - 1)
    Am = _csr_dev(rp, col, val)
    xd = dev(x)
    ref = O.spmv_csr(rp.astype(np.int32), col.astype(np.int32), val, x)
    cc.l2_persist(xd, 1.0)
    try:
        for v in (dict(backend="default"), dict(backend="agent", order="row")):
            y = ops.spmv(Am, xd, **v)
            torch.cuda.synchronize()
            got = y.cpu().numpy()
            nz = ref != 0
            assert relerr(got[nz], ref[nz]) <= TOL
    finally:
        cc.l2_persist(None)
    with pytest.raises(cc.CtaclustError):
        cc.l2_persist(xd, 0.0)
