"""CPU oracle for libctaclust.

TEST INFRASTRUCTURE ONLY -- only ``tests/``, ``__graft_entry__.smoke()`` and the
``cpu_baseline`` / ``--impl reference`` legs of ``bench.py`` may import, call,
link or execute anything under ``oracle/``.  The product path
(``paper_conf_asplos_lis0l0c17_b200``) never imports it and shares no code with
it.  The C definitions live in ``oracle/oracle.c`` (fp64 accumulation); this
module only marshals numpy arrays into them.  ``oracle/plan.py`` is the
schedule oracle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import plan  # noqa: F401  (re-export)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


_LIB_OMP = os.path.join(_HERE, "liboracle_omp.so")
_omp = False


def build(force: bool = False, omp: bool = False) -> str:
    """Compile oracle.c with plain gcc -O2 (no -ffast-math: keep IEEE order).
    omp=True: the same source with -fopenmp (all-core timing only)."""
    lib = _LIB_OMP if omp else _LIB
    if force or not os.path.exists(lib) or os.path.getmtime(lib) < os.path.getmtime(_SRC):
        flags = ["-fopenmp"] if omp else []
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-std=c11"] + flags +
                              ["-o", lib + ".tmp", _SRC])
        os.replace(lib + ".tmp", lib)
    return lib


def use_openmp(on: bool = True) -> None:
    """Route the wrappers below to the OpenMP build (bench.py cpu_baseline's
    all-core leg) or back to the plain serial build."""
    global _lib, _omp
    if on != _omp:
        _omp, _lib = on, None


def omp_threads() -> int:
    """Threads the OpenMP build uses (omp_get_max_threads), 1 for the plain build."""
    if not _omp:
        return 1
    try:
        return int(ctypes.CDLL(build(omp=True)).omp_get_max_threads())
    except AttributeError:
        g = ctypes.CDLL("libgomp.so.1")
        return int(g.omp_get_max_threads())


def _load():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build(omp=_omp))
    return _lib


def _f32(a):
    a = np.ascontiguousarray(a, dtype=np.float32)
    return a, a.ctypes.data_as(ctypes.c_void_p)


def _i32(a):
    a = np.ascontiguousarray(a, dtype=np.int32)
    return a, a.ctypes.data_as(ctypes.c_void_p)


def _out(n):
    o = np.zeros(n, dtype=np.float64)
    return o, o.ctypes.data_as(ctypes.c_void_p)


_I = ctypes.c_int64


def _mat(A):
    A = np.asarray(A, dtype=np.float32)
    m, n = A.shape
    lda = A.strides[0] // 4 if A.flags["C_CONTIGUOUS"] else n
    A = np.ascontiguousarray(A)
    return A, m, n, n, A.ctypes.data_as(ctypes.c_void_p)


def matvec(A, x):
    A, m, n, lda, pA = _mat(A)
    x, px = _f32(x)
    y, py = _out(m)
    _load().oracle_matvec(_I(m), _I(n), pA, _I(lda), px, py)
    return y


def atax(A, x):
    A, m, n, lda, pA = _mat(A)
    x, px = _f32(x)
    tmp, pt = _out(m)
    y, py = _out(n)
    _load().oracle_atax(_I(m), _I(n), pA, _I(lda), px, pt, py)
    return tmp, y


def atax_pass2(A, tmp32):
    A, m, n, lda, pA = _mat(A)
    t, pt = _f32(tmp32)
    y, py = _out(n)
    _load().oracle_atax_pass2(_I(m), _I(n), pA, _I(lda), pt, py)
    return y


def bicg(A, p, r):
    A, m, n, lda, pA = _mat(A)
    p, pp = _f32(p)
    r, pr = _f32(r)
    q, pq = _out(m)
    s, ps = _out(n)
    _load().oracle_bicg(_I(m), _I(n), pA, _I(lda), pp, pr, pq, ps)
    return q, s


def mvt(A, x1, x2, y1, y2):
    A, m, n, lda, pA = _mat(A)
    x1, p1 = _f32(x1)
    x2, p2 = _f32(x2)
    y1, p3 = _f32(y1)
    y2, p4 = _f32(y2)
    o1, q1 = _out(m)
    o2, q2 = _out(n)
    _load().oracle_mvt(_I(m), _I(n), pA, _I(lda), p1, p2, p3, p4, q1, q2)
    return o1, o2


def jacobi5(u0, iters):
    u0 = np.ascontiguousarray(u0, dtype=np.float32)
    rows, cols = u0.shape
    out = np.zeros((rows, cols), dtype=np.float64)
    work = np.zeros(2 * rows * cols, dtype=np.float64)
    _load().oracle_jacobi5(_I(rows), _I(cols), u0.ctypes.data_as(ctypes.c_void_p),
                           ctypes.c_int(iters), out.ctypes.data_as(ctypes.c_void_p),
                           work.ctypes.data_as(ctypes.c_void_p))
    return out


def jacobi5_f32(u0, iters):
    u0 = np.ascontiguousarray(u0, dtype=np.float32)
    rows, cols = u0.shape
    out = np.zeros((rows, cols), dtype=np.float32)
    work = np.zeros(2 * rows * cols, dtype=np.float32)
    _load().oracle_jacobi5_f32(_I(rows), _I(cols), u0.ctypes.data_as(ctypes.c_void_p),
                               ctypes.c_int(iters), out.ctypes.data_as(ctypes.c_void_p),
                               work.ctypes.data_as(ctypes.c_void_p))
    return out


def conv2d(img, w):
    img = np.ascontiguousarray(img, dtype=np.float32)
    w = np.ascontiguousarray(w, dtype=np.float32)
    K = w.shape[0]
    assert w.shape == (K, K) and K % 2 == 1
    rows, cols = img.shape
    out = np.zeros((rows, cols), dtype=np.float64)
    _load().oracle_conv2d(_I(rows), _I(cols), img.ctypes.data_as(ctypes.c_void_p),
                          ctypes.c_int(K // 2), w.ctypes.data_as(ctypes.c_void_p),
                          out.ctypes.data_as(ctypes.c_void_p))
    return out


def spmv_csr(row_ptr, col, val, x):
    rp, prp = _i32(row_ptr)
    c, pc = _i32(col)
    v, pv = _f32(val)
    x, px = _f32(x)
    rows = len(rp) - 1
    y, py = _out(rows)
    _load().oracle_spmv_csr(_I(rows), prp, pc, pv, px, py)
    return y


def hist64(data):
    """64-bin histogram of uint8 data (bin = byte >> 2); uint64 counts."""
    data = np.ascontiguousarray(data, dtype=np.uint8)
    out = np.zeros(64, dtype=np.uint64)
    _load().oracle_hist64(ctypes.c_int64(data.size), data.ctypes.data_as(ctypes.c_void_p),
                          out.ctypes.data_as(ctypes.c_void_p))
    return out
