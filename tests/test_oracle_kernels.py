"""Pins for the C kernel oracle (oracle/oracle.c) against closed forms, special
cases and independent library routines (numpy / scipy), on non-square and
ragged shapes so that a transposed operand, a dropped term or a wrong index
fails.  None of these compares the oracle with itself."""
import numpy as np
import pytest
import scipy.signal
import scipy.sparse

import oracle as O
from paper_conf_asplos_lis0l0c17_b200 import synth


@pytest.fixture(scope="module", autouse=True)
def _build():
    O.build()


def rnd(seed, *shape):
    return synth.uniform(seed, int(np.prod(shape))).reshape(shape)


# ---- matvec (Listing 1/2) ----
def test_matvec_identity_and_ones():
    n = 37
    x = rnd(1, n)
    assert np.array_equal(O.matvec(np.eye(n, dtype=np.float32), x), x.astype(np.float64))
    assert np.array_equal(O.matvec(np.ones((5, 300), np.float32), np.ones(300, np.float32)),
                          np.full(5, 300.0))


@pytest.mark.parametrize("m,n", [(1, 1), (33, 70), (70, 33), (128, 1000)])
def test_matvec_vs_numpy(m, n):
    A, x = rnd(2, m, n), rnd(3, n)
    ref = A.astype(np.float64) @ x.astype(np.float64)
    assert np.allclose(O.matvec(A, x), ref, rtol=1e-13, atol=0)


# ---- ATAX / BICG / MVT (Table 2, PolyBench definitions) ----
@pytest.mark.parametrize("m,n", [(1, 1), (45, 19), (19, 45), (64, 300)])
def test_atax_bicg_mvt_vs_numpy(m, n):
    A = rnd(4, m, n).astype(np.float64)
    x, p, r = rnd(5, n), rnd(6, n), rnd(7, m)
    x1, x2, y1, y2 = rnd(8, m), rnd(9, n), rnd(10, n), rnd(11, m)
    tmp, y = O.atax(A, x)
    assert np.allclose(tmp, A @ x, rtol=1e-13) and np.allclose(y, A.T @ (A @ x), rtol=1e-13)
    q, s = O.bicg(A, p, r)
    assert np.allclose(q, A @ p, rtol=1e-13) and np.allclose(s, A.T @ r, rtol=1e-13)
    o1, o2 = O.mvt(A, x1, x2, y1, y2)
    assert np.allclose(o1, x1 + A @ y1, rtol=1e-13) and np.allclose(o2, x2 + A.T @ y2, rtol=1e-13)
    t32 = tmp.astype(np.float32)
    assert np.allclose(O.atax_pass2(A, t32), A.T @ t32.astype(np.float64), rtol=1e-13)


def test_atax_identity():
    n = 50
    x = rnd(12, n)
    tmp, y = O.atax(np.eye(n, dtype=np.float32), x)
    assert np.array_equal(y, x.astype(np.float64)) and np.array_equal(tmp, y)


def test_integer_exact_mode_is_exact():
    # integer inputs in {-8..8}: all partial sums < 2^24, so fp64 == exact integer math
    m, n = 40, 70
    A = synth.small_int(13, m * n).reshape(m, n)
    p, r = synth.small_int(14, n), synth.small_int(15, m)
    q, s = O.bicg(A, p, r)
    Ai = A.astype(np.int64)
    assert np.array_equal(q, (Ai @ p.astype(np.int64)).astype(np.float64))
    assert np.array_equal(s, (Ai.T @ r.astype(np.int64)).astype(np.float64))


# ---- Jacobi 5-point ----
def test_jacobi_constant_is_fixed_point():
    u = np.full((9, 13), 3.25, np.float32)
    assert np.allclose(O.jacobi5(u, 7), 3.25, rtol=0, atol=1e-12)


def test_jacobi_linear_field_is_harmonic():
    i, j = np.meshgrid(np.arange(11), np.arange(17), indexing="ij")
    u = (0.25 * i + 0.125 * j + 1.0).astype(np.float32)
    assert np.allclose(O.jacobi5(u, 25), u, rtol=0, atol=1e-12)


@pytest.mark.parametrize("p,q,t", [(1, 1, 1), (2, 3, 5), (3, 1, 20)])
def test_jacobi_eigenmode_closed_form(p, q, t):
    """u = sin(pi p i/(R-1)) sin(pi q j/(C-1)) vanishes on the boundary and is an
    eigenvector of the Jacobi sweep with eigenvalue
    0.2 * (1 + 2 cos(pi p/(R-1)) + 2 cos(pi q/(C-1)))."""
    R, C = 13, 21
    i, j = np.meshgrid(np.arange(R), np.arange(C), indexing="ij")
    u64 = np.sin(np.pi * p * i / (R - 1)) * np.sin(np.pi * q * j / (C - 1))
    u = u64.astype(np.float32)
    lam = 0.2 * (1 + 2 * np.cos(np.pi * p / (R - 1)) + 2 * np.cos(np.pi * q / (C - 1)))
    got = O.jacobi5(u, t)
    # the fp32-rounded start is an eigenvector up to 6e-8 relative
    assert np.allclose(got, lam ** t * u64, rtol=0, atol=2e-7)


# ---- fp32 Jacobi (the bit-exact reference of the GPU sweep) ----
# Pins written as functions of the routine under test so that
# tests/test_oracle_mutants.py can run them against deliberately broken
# builds of oracle.c and show that each plausible mistake fails one of them.
def pin_jacobi_f32_tracks_fp64(f32):
    """fp32 sweeps stay within a few ulp of the fp64 definition on U[0,1)
    fields (no cancellation: every term is positive).  A dropped, duplicated
    or mis-indexed neighbour moves results by ~20 %, far above 1e-6."""
    for it in (1, 3, 7):
        u = rnd(31, 37, 53)
        ref = O.jacobi5(u, it)
        got = f32(u, it).astype(np.float64)
        assert np.max(np.abs(got - ref) / np.abs(ref)) <= 1e-6, it


def pin_jacobi_f32_eigenmode(f32):
    """The separable sine mode decays by its closed-form eigenvalue in fp32 too."""
    R, C = 13, 21
    i, j = np.meshgrid(np.arange(R), np.arange(C), indexing="ij")
    for p, q, t in ((1, 1, 1), (2, 3, 5), (3, 1, 20)):
        u64 = np.sin(np.pi * p * i / (R - 1)) * np.sin(np.pi * q * j / (C - 1))
        lam = 0.2 * (1 + 2 * np.cos(np.pi * p / (R - 1)) + 2 * np.cos(np.pi * q / (C - 1)))
        assert np.max(np.abs(f32(u64.astype(np.float32), t) - lam ** t * u64)) <= 5e-7, (p, q, t)


def pin_jacobi_f32_by_hand(f32):
    """3x3 grids: only the centre moves.  (a) arange: 0.2f*(4+3+5+7+1) = 0.2f*20
    rounds to 4.0.  (b) the PolyBench sum order, by hand: with c = 2^24,
    w = e = n = 1 and s = -2^24, ((((c+w)+e)+s)+n) in fp32 is
    2^24 -> 2^24 (ties to even) -> 0 -> 1, so the centre becomes 0.2f; adding
    n before s would give 0, the exact sum 3 would give 0.6."""
    u = np.arange(9, dtype=np.float32).reshape(3, 3)
    want = u.copy()
    want[1, 1] = 4.0
    assert np.array_equal(f32(u, 1), want)
    v = np.zeros((3, 3), np.float32)
    v[1, 1], v[1, 0], v[1, 2], v[2, 1], v[0, 1] = 2.0 ** 24, 1, 1, -(2.0 ** 24), 1
    got = f32(v, 1)
    assert got[1, 1] == np.float32(0.2)
    want = v.copy()
    want[1, 1] = np.float32(0.2)
    assert np.array_equal(got, want)


def pin_jacobi_f32_fixed_points(f32):
    for c in (1.0, 0.5, 2.0, 0.25):                       # 0.2f*5c rounds to c
        assert np.array_equal(f32(np.full((6, 7), c, np.float32), 3), np.full((6, 7), c, np.float32))


JACOBI_F32_PINS = [pin_jacobi_f32_tracks_fp64, pin_jacobi_f32_eigenmode, pin_jacobi_f32_by_hand,
                   pin_jacobi_f32_fixed_points]


@pytest.mark.parametrize("pin", JACOBI_F32_PINS, ids=lambda f: f.__name__)
def test_jacobi_f32_pins(pin):
    pin(O.jacobi5_f32)


def test_jacobi_single_sweep_tiny_by_hand():
    u = np.arange(9, dtype=np.float32).reshape(3, 3)
    got = O.jacobi5(u, 1)
    expect = u.astype(np.float64).copy()
    expect[1, 1] = 0.2 * (4 + 3 + 5 + 1 + 7)                # centre and its four neighbours
    assert np.array_equal(got, expect)


# ---- conv2d (cross-correlation, interior only) ----
@pytest.mark.parametrize("R", [1, 3])
def test_conv_vs_scipy_correlate(R):
    img = rnd(16, 40, 53)
    w = rnd(17, 2 * R + 1, 2 * R + 1)                        # asymmetric: catches a flip
    got = O.conv2d(img, w)
    ref = scipy.signal.correlate2d(img.astype(np.float64), w.astype(np.float64), mode="valid")
    assert np.allclose(got[R:-R, R:-R], ref, rtol=1e-13)
    border = got.copy()
    border[R:-R, R:-R] = 0
    assert not border.any()


def test_conv_delta_and_ones():
    img = rnd(18, 20, 30)
    d = np.zeros((7, 7), np.float32)
    d[3, 3] = 1
    assert np.array_equal(O.conv2d(img, d)[3:-3, 3:-3], img[3:-3, 3:-3].astype(np.float64))
    assert np.array_equal(O.conv2d(np.ones((8, 9), np.float32), np.ones((3, 3), np.float32))[1:-1, 1:-1],
                          np.full((6, 7), 9.0))


# ---- CSR SpMV ----
def test_spmv_vs_scipy():
    rp, col = synth.rmat_csr(19, 9, 8)
    val = rnd(20, len(col))
    x = rnd(21, len(rp) - 1)
    n = len(rp) - 1
    ref = scipy.sparse.csr_matrix((val.astype(np.float64), col, rp), shape=(n, n)) @ x.astype(np.float64)
    assert np.allclose(O.spmv_csr(rp, col, val, x), ref, rtol=1e-13)


def test_spmv_identity_and_permutation():
    n = 100
    x = rnd(22, n)
    rp = np.arange(n + 1, dtype=np.int32)
    assert np.array_equal(O.spmv_csr(rp, np.arange(n, dtype=np.int32), np.ones(n, np.float32), x),
                          x.astype(np.float64))
    perm = synth.random_permutation(3, n).astype(np.int32)
    assert np.array_equal(O.spmv_csr(rp, perm, np.ones(n, np.float32), x), x[perm].astype(np.float64))


def test_rmat_generator_shape():
    rp, col = synth.rmat_csr(23, 10, 16)
    n = 1 << 10
    assert rp[0] == 0 and len(rp) == n + 1 and rp[-1] == len(col)
    assert np.all(np.diff(rp) >= 0) and col.min() >= 0 and col.max() < n
    for i in range(0, n, 97):                               # sorted, no duplicates
        c = col[rp[i]:rp[i + 1]]
        assert np.all(np.diff(c) > 0)
    deg = np.diff(rp)
    assert deg.max() > 8 * deg.mean()                       # power-law: heavy head


def test_synth_numpy_torch_identical():
    import torch
    a = synth.uniform(5, 1000, 12345)
    b = synth.uniform(5, 1000, 12345, backend="torch").numpy()
    assert np.array_equal(a, b)
    c = synth.small_int(6, 1000, 7)
    d = synth.small_int(6, 1000, 7, backend="torch").numpy()
    assert np.array_equal(c, d)
    big = synth.uniform(1, 10, (1 << 33) + 5)               # high index word matters
    assert not np.array_equal(big, synth.uniform(1, 10, 5))
    assert torch.is_tensor(synth.uniform(1, 4, backend="torch"))


# ---- S8(f)3 64-bin histogram (Table 2; reading R24: bin = byte >> 2) ----
def test_hist64_closed_forms():
    # every byte value r times: each bin holds its 4 byte values -> 4r
    r = 37
    counts = O.hist64(np.tile(np.arange(256, dtype=np.uint8), r))
    assert counts.dtype == np.uint64 and counts.shape == (64,)
    assert np.all(counts == 4 * r)
    # a constant input lands in one bin: byte c -> bin floor(c / 4)
    for c in (0, 3, 4, 130, 255):
        counts = O.hist64(np.full(1001, c, dtype=np.uint8))
        assert counts[c // 4] == 1001 and counts.sum() == 1001
    assert np.all(O.hist64(np.zeros(0, dtype=np.uint8)) == 0)


def test_hist64_threshold_counts_and_total():
    # prefix sums of the histogram count the bytes below each bin edge 4k
    for kind in ("uniform", "skewed"):
        data = synth.bytes_u8(21, 100003, kind=kind)
        counts = O.hist64(data)
        assert int(counts.sum()) == data.size
        cum = np.concatenate([[0], np.cumsum(counts)])
        for k in range(65):
            assert cum[k] == np.count_nonzero(data < 4 * k)


def test_bytes_generator_backends_agree_and_skew():
    import torch
    a = synth.bytes_u8(5, 70001, kind="skewed")
    b = synth.bytes_u8(5, 70001, kind="skewed", backend="torch").numpy()
    assert np.array_equal(a, b)
    frac0 = np.count_nonzero(a < 4) / a.size            # 3/4 hot + 1/4 * 4/256 uniform
    assert abs(frac0 - (0.75 + 0.25 * 4 / 256)) < 0.01
    u = synth.bytes_u8(6, 1 << 16)
    assert abs(np.count_nonzero(u < 128) / u.size - 0.5) < 0.01
