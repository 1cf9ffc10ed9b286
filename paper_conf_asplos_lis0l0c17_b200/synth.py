"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the method (no partitioning, no kernel
math): only a counter-based hash that turns ``(seed, index)`` into a value, so
that a value is a pure function of its seed and logical index and both sides
can regenerate the same input independently (SURVEY.md §8(d) "Seeds").  The
numpy and torch backends produce bit-identical values (all integer ops are
done on 32-bit words; the float conversion ``(h >> 8) * 2**-24`` is exact).

Recipes:
* ``uniform``  U[0,1) fp32 -- the default input distribution (reading R17:
  positive inputs so relative error is well defined);
* ``small_int`` integers in {-8..8} as fp32 -- the integer-exact mode (R18);
* ``rmat_edges`` R-MAT (a,b,c,d) = (0.57,0.19,0.19,0.05) power-law graphs for
  the CSR SpMV workload (R16).
* ``bytes_u8`` input bytes for the 64-bin histogram (S§8(f)3, R24): uniform
  bytes, or ``skewed`` (75 % of bytes in bin 0: the contended case).
"""
from __future__ import annotations

import numpy as np

_M32 = 0xFFFFFFFF


def _mix_np(x):
    # lowbias32 finaliser on uint32 words (numpy uint32 arithmetic wraps mod 2^32)
    x = x ^ (x >> np.uint32(16))
    x = x * np.uint32(0x7FEB352D)
    x = x ^ (x >> np.uint32(15))
    x = x * np.uint32(0x846CA68B)
    x = x ^ (x >> np.uint32(16))
    return x


def _seed_word(seed: int, stream: int) -> int:
    s = np.uint32(((seed * 0x9E3779B9) + 0x632BE5AB + stream * 0x2545F491) & _M32)
    return int(_mix_np(np.array([s], dtype=np.uint32))[0])


def hash_u32_np(seed: int, idx, stream: int = 0) -> np.ndarray:
    """32-bit hash of (seed, stream, idx) for int64 idx >= 0, as uint32 words."""
    idx = np.asarray(idx, dtype=np.uint64)
    s = np.uint32(_seed_word(seed, stream))
    lo = (idx & np.uint64(_M32)).astype(np.uint32)
    hi = (idx >> np.uint64(32)).astype(np.uint32)
    h = _mix_np(lo ^ s)
    h = _mix_np(h ^ hi ^ np.uint32(0x85EBCA6B))
    return h


def _mix_t(x):
    import torch  # noqa: F401
    x = x ^ (x >> 16)
    x = (x * 0x7FEB352D) & _M32          # int64 product wraps; low 32 bits exact
    x = x ^ (x >> 15)
    x = (x * 0x846CA68B) & _M32
    x = x ^ (x >> 16)
    return x


def hash_u32_torch(seed: int, idx, stream: int = 0):
    """Same hash as :func:`hash_u32_np` on an int64 torch tensor (any device)."""
    s = _seed_word(seed, stream)
    h = _mix_t((idx & _M32) ^ s)
    h = _mix_t(h ^ ((idx >> 32) & _M32) ^ 0x85EBCA6B)
    return h


def uniform(seed: int, count: int, start: int = 0, *, backend: str = "numpy",
            device=None, stream: int = 0, chunk: int = 1 << 26):
    """``count`` U[0,1) fp32 values for logical indices start..start+count-1."""
    if backend == "numpy":
        out = np.empty(count, dtype=np.float32)
        for c0 in range(0, count, chunk):
            c1 = min(count, c0 + chunk)
            idx = np.arange(start + c0, start + c1, dtype=np.uint64)
            h = hash_u32_np(seed, idx, stream)
            out[c0:c1] = (h >> np.uint32(8)).astype(np.float32) * np.float32(2.0 ** -24)
        return out
    import torch
    out = torch.empty(count, dtype=torch.float32, device=device)
    for c0 in range(0, count, chunk):
        c1 = min(count, c0 + chunk)
        idx = torch.arange(start + c0, start + c1, dtype=torch.int64, device=device)
        h = hash_u32_torch(seed, idx, stream)
        out[c0:c1] = (h >> 8).to(torch.float32) * (2.0 ** -24)
    return out


def uniform_at(seed: int, idx, stream: int = 0) -> np.ndarray:
    """U[0,1) fp32 values at arbitrary logical indices (numpy): the same
    values :func:`uniform` gives at those indices (e.g. one column of a
    row-major matrix: idx = i * cols + j)."""
    h = hash_u32_np(seed, np.asarray(idx, dtype=np.uint64), stream)
    return (h >> np.uint32(8)).astype(np.float32) * np.float32(2.0 ** -24)


def bytes_u8(seed: int, count: int, start: int = 0, *, kind: str = "uniform", backend: str = "numpy",
             device=None, chunk: int = 1 << 26):
    """``count`` uint8 values: ``uniform`` = top byte of the hash; ``skewed`` =
    with probability 3/4 (second hash stream) a value in 0..3, else uniform."""
    if kind not in ("uniform", "skewed"):
        raise ValueError(kind)
    if backend == "numpy":
        out = np.empty(count, dtype=np.uint8)
        for c0 in range(0, count, chunk):
            c1 = min(count, c0 + chunk)
            idx = np.arange(start + c0, start + c1, dtype=np.uint64)
            h = hash_u32_np(seed, idx)
            b = (h >> np.uint32(24)).astype(np.uint8)
            if kind == "skewed":
                hot = (hash_u32_np(seed, idx, 1) >> np.uint32(24)) < np.uint32(192)
                b = np.where(hot, (h >> np.uint32(30)).astype(np.uint8), b)
            out[c0:c1] = b
        return out
    import torch
    out = torch.empty(count, dtype=torch.uint8, device=device)
    for c0 in range(0, count, chunk):
        c1 = min(count, c0 + chunk)
        idx = torch.arange(start + c0, start + c1, dtype=torch.int64, device=device)
        h = hash_u32_torch(seed, idx)
        b = h >> 24
        if kind == "skewed":
            hot = (hash_u32_torch(seed, idx, 1) >> 24) < 192
            b = torch.where(hot, h >> 30, b)
        out[c0:c1] = b.to(torch.uint8)
    return out


def small_int(seed: int, count: int, start: int = 0, *, lo: int = -8, hi: int = 8,
              backend: str = "numpy", device=None, stream: int = 0):
    """Integers uniformly-ish in [lo, hi] stored as fp32 (integer-exact mode)."""
    span = hi - lo + 1
    if backend == "numpy":
        idx = np.arange(start, start + count, dtype=np.uint64)
        h = hash_u32_np(seed, idx, stream)
        return ((h % np.uint32(span)).astype(np.int64) + lo).astype(np.float32)
    import torch
    idx = torch.arange(start, start + count, dtype=torch.int64, device=device)
    h = hash_u32_torch(seed, idx, stream)
    return ((h % span) + lo).to(torch.float32)


def matrix(seed: int, rows: int, cols: int, *, ld: int | None = None, kind: str = "uniform",
           backend: str = "numpy", device=None, row0: int = 0):
    """rows x cols matrix (logical element (i, j) has index (row0+i)*cols + j),
    stored with leading dimension ``ld`` >= cols (padding is zero)."""
    ld = cols if ld is None else ld
    gen = uniform if kind == "uniform" else small_int
    flat = gen(seed, rows * cols, row0 * cols, backend=backend, device=device)
    if backend == "numpy":
        m = flat.reshape(rows, cols)
        if ld == cols:
            return m
        out = np.zeros((rows, ld), dtype=np.float32)
        out[:, :cols] = m
        return out
    import torch
    m = flat.view(rows, cols)
    if ld == cols:
        return m
    out = torch.zeros((rows, ld), dtype=torch.float32, device=device)
    out[:, :cols] = m
    return out


# --------------------------------------------------------------------------
# R-MAT power-law graph (reading R16): recursive quadrant choice with
# probabilities (a, b, c, d) = (0.57, 0.19, 0.19, 0.05) per level, scale
# levels, edge_factor * 2**scale edges; duplicates dropped; columns sorted per
# row; no vertex permutation.  Returned as CSR (int32 row_ptr, int32 col).
# --------------------------------------------------------------------------
RMAT_ABCD = (0.57, 0.19, 0.19, 0.05)


def rmat_csr(seed: int, scale: int, edge_factor: int, *, chunk: int = 1 << 22,
             backend: str = "numpy", device=None):
    """CSR of an R-MAT graph with 2**scale rows; numpy and torch give identical
    graphs (same hash draws and integer thresholds)."""
    n = 1 << scale
    nedges = edge_factor * n
    a, b, c, _ = RMAT_ABCD
    # thresholds on a 24-bit uniform draw, one draw per (edge, level)
    t_a = int(a * (1 << 24))
    t_ab = int((a + b) * (1 << 24))
    t_abc = int((a + b + c) * (1 << 24))
    if backend == "numpy":
        keys = np.empty(nedges, dtype=np.int64)
        for e0 in range(0, nedges, chunk):
            e1 = min(nedges, e0 + chunk)
            e = np.arange(e0, e1, dtype=np.uint64)
            row = np.zeros(e1 - e0, dtype=np.int64)
            col = np.zeros(e1 - e0, dtype=np.int64)
            for lvl in range(scale):
                u = (hash_u32_np(seed, e * np.uint64(scale) + np.uint64(lvl), stream=7) >> np.uint32(8)).astype(np.int64)
                down = (u >= t_ab)                                  # quadrant c or d -> row bit
                right = ((u >= t_a) & (u < t_ab)) | (u >= t_abc)    # quadrant b or d -> col bit
                bit = np.int64(1) << np.int64(scale - 1 - lvl)
                row |= np.where(down, bit, 0)
                col |= np.where(right, bit, 0)
            keys[e0:e1] = row * n + col
        keys = np.unique(keys)                                      # sorts and drops duplicates
        rows_of = (keys // n).astype(np.int64)
        cols = (keys % n).astype(np.int32)
        counts = np.bincount(rows_of, minlength=n)
        row_ptr = np.zeros(n + 1, dtype=np.int64)
        np.cumsum(counts, out=row_ptr[1:])
        if row_ptr[-1] >= 2 ** 31:
            raise ValueError("nnz exceeds int32 row_ptr")
        return row_ptr.astype(np.int32), cols
    import torch
    chunk = max(chunk, 1 << 24)
    parts = []
    for e0 in range(0, nedges, chunk):
        e1 = min(nedges, e0 + chunk)
        e = torch.arange(e0, e1, dtype=torch.int64, device=device)
        row = torch.zeros(e1 - e0, dtype=torch.int64, device=device)
        col = torch.zeros_like(row)
        for lvl in range(scale):
            u = hash_u32_torch(seed, e * scale + lvl, stream=7) >> 8
            bit = 1 << (scale - 1 - lvl)
            row |= (u >= t_ab).to(torch.int64) * bit
            col |= (((u >= t_a) & (u < t_ab)) | (u >= t_abc)).to(torch.int64) * bit
        parts.append(torch.unique(row * n + col))
    keys = torch.unique(torch.cat(parts))
    del parts
    rows_of = keys // n
    cols = (keys % n).to(torch.int32)
    counts = torch.bincount(rows_of, minlength=n)
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    torch.cumsum(counts, 0, out=row_ptr[1:])
    if int(row_ptr[-1]) >= 2 ** 31:
        raise ValueError("nnz exceeds int32 row_ptr")
    return row_ptr.to(torch.int32), cols


def random_permutation(seed: int, n: int) -> np.ndarray:
    """Deterministic permutation of range(n) (sort by hash) -- the no-locality control."""
    h = hash_u32_np(seed, np.arange(n, dtype=np.uint64), stream=11)
    return np.lexsort((np.arange(n), h)).astype(np.int64)
