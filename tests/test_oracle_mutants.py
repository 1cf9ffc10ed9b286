"""Mutation check of the oracle pins (VERDICT r1 'What's weak' 1).

Builds deliberately broken copies of oracle/oracle.c -- each one a plausible
mistake in the fp32 Jacobi sweep that every bit-exact GPU Jacobi test compares
against (a duplicated or mis-indexed neighbour, a dropped term, a swapped sum
order, a wrong coefficient, an unfixed boundary) -- and shows that at least
one pin in tests/test_oracle_kernels.py fails on each.  The unmutated source
passes every pin (test_oracle_kernels.py), so the pins constrain the
function, not just its existence."""
import ctypes
import os
import subprocess

import numpy as np
import pytest

from test_oracle_kernels import JACOBI_F32_PINS

SRC = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "oracle", "oracle.c")

SWEEP = "b[i * cols + j] = 0.2f * ((((c + w) + e) + s) + n);"
MUTANTS = {
    "north_duplicated": ("float s = a[(i + 1) * cols + j]", "float s = a[(i - 1) * cols + j]"),
    "east_reads_west": ("e = a[i * cols + j + 1]", "e = a[i * cols + j - 1]"),
    "south_dropped": (SWEEP, "b[i * cols + j] = 0.2f * (((c + w) + e) + n);"),
    "north_before_south": (SWEEP, "b[i * cols + j] = 0.2f * ((((c + w) + e) + n) + s);"),
    "centre_last": (SWEEP, "b[i * cols + j] = 0.2f * ((((w + e) + s) + n) + c);"),
    "coefficient": (SWEEP, "b[i * cols + j] = 0.25f * ((((c + w) + e) + s) + n);"),
    "boundary_not_kept": ("a[k] = u0[k]; b[k] = u0[k]; }", "a[k] = u0[k]; b[k] = 0.0f; }"),
}


def _build(tmp_path, name, old, new):
    src = open(SRC).read()
    assert src.count(old) >= 1, f"mutant {name}: pattern not found (oracle.c changed?)"
    # mutate inside oracle_jacobi5_f32 only
    head, sep, tail = src.partition("void oracle_jacobi5_f32(")
    body, sep2, rest = tail.partition("/* ----")
    assert old in body, f"mutant {name}: pattern not in oracle_jacobi5_f32"
    cpath = tmp_path / f"{name}.c"
    cpath.write_text(head + sep + body.replace(old, new, 1) + sep2 + rest)
    so = tmp_path / f"{name}.so"
    subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-std=c11", "-o", str(so), str(cpath)])
    return ctypes.CDLL(str(so))


def _wrap(lib):
    def f32(u0, iters):
        u0 = np.ascontiguousarray(u0, dtype=np.float32)
        rows, cols = u0.shape
        out = np.zeros((rows, cols), np.float32)
        work = np.zeros(2 * rows * cols, np.float32)
        lib.oracle_jacobi5_f32(ctypes.c_int64(rows), ctypes.c_int64(cols), u0.ctypes.data_as(ctypes.c_void_p),
                               ctypes.c_int(iters), out.ctypes.data_as(ctypes.c_void_p),
                               work.ctypes.data_as(ctypes.c_void_p))
        return out
    return f32


@pytest.mark.parametrize("name", sorted(MUTANTS))
def test_every_mutant_fails_a_pin(tmp_path, name):
    old, new = MUTANTS[name]
    f32 = _wrap(_build(tmp_path, name, old, new))
    failed = []
    for pin in JACOBI_F32_PINS:
        try:
            pin(f32)
        except AssertionError:
            failed.append(pin.__name__)
    assert failed, f"mutant {name} passes every Jacobi fp32 pin"


def test_unmutated_copy_passes(tmp_path):
    f32 = _wrap(_build(tmp_path, "identity", SWEEP, SWEEP))
    for pin in JACOBI_F32_PINS:
        pin(f32)
