"""Tensor-level entry points over the C ABI (what tests, bench and users call).

Each function allocates outputs with torch on the inputs' device, builds (and
caches) the cluster plan for the kernel's logical grid, and issues one
``cc_launch``.  No arithmetic of the method happens here.
"""
from __future__ import annotations

import torch

from . import ctaclust as cc

# default partition per kernel: the ATAX family is X-P (column-major
# indexing, "X-P" for ATX/MVT/BC in Table 2); matvec is
# row-clustered per config 1.  For the stencils the paper's tile-wise order
# (Fig. 7) is available, but on B200 the row-major (Y-P) partition measures
# fastest with TMA staging, so it is the default here.
DEFAULT_ORDER = {"census": ("row", (1, 1)), "matvec": ("row", (1, 1)), "atax": ("col", (1, 1)),
                 "bicg": ("col", (1, 1)), "mvt": ("col", (1, 1)), "jacobi5": ("row", (1, 1)),
                 "conv2d": ("row", (1, 1)), "spmv": ("row", (1, 1)), "hist64": ("row", (1, 1)),
                 "jacobi5_halo": ("row", (1, 1)), "atax_fused": ("row", (1, 1)), "spmv_shub": ("row", (1, 1)),
                 "jacobi5_wave": ("col", (1, 1))}

# Plans of the computed orders are cached for the life of the process: a plan
# may only be destroyed once every stream that used it has synchronized
# (cc_plan_destroy), which a cache cannot know.  Call release_plans() to drop
# them.  USER-order plans are keyed by the order table's content (a hash) and
# kept in a small LRU; an evicted one is destroyed only after synchronizing
# its device.
_plans: dict = {}
_user_plans: "OrderedDict" = None
USER_PLAN_CACHE = 8


def release_plans() -> None:
    """Synchronize every device holding a cached plan and drop them all (frees
    their device tables and workspaces)."""
    devs = {p.device for p in _plans.values()} | {p.device for p in (_user_plans or {}).values()}
    for d in devs:
        if d is not None and d >= 0:
            torch.cuda.synchronize(d)
    _plans.clear()
    if _user_plans is not None:
        _user_plans.clear()


def _user_plan(gx, gy, user_order, num_clusters, device) -> cc.Plan:
    import hashlib
    from collections import OrderedDict

    import numpy as np
    global _user_plans
    if _user_plans is None:
        _user_plans = OrderedDict()
    arr = np.ascontiguousarray(user_order, dtype=np.int32)
    key = (gx, gy, hashlib.blake2b(arr.tobytes(), digest_size=16).digest(), num_clusters, device)
    p = _user_plans.get(key)
    if p is not None:
        _user_plans.move_to_end(key)
        return p
    p = cc.Plan(gx, gy, "user", num_clusters, user_order=arr, device=device)
    _user_plans[key] = p
    while len(_user_plans) > USER_PLAN_CACHE:
        _, old = _user_plans.popitem(last=False)
        if old.device is not None and old.device >= 0:
            torch.cuda.synchronize(old.device)          # no stream may still use it
        old.close()
    return p


def plan_for(kernel: str, args, order=None, tile=None, num_clusters: int = 0, device: int = 0,
             user_order=None) -> cc.Plan:
    gx, gy = cc.kernel_grid(kernel, args)
    o, t = DEFAULT_ORDER[kernel]
    order = o if order is None else order
    tile = t if tile is None else tile
    if user_order is not None:
        # keyed by content; a per-call hash of the table costs host time
        # (~0.1 ms per 256 KB), so hot loops should pass a Plan to cc.launch
        return _user_plan(gx, gy, user_order, num_clusters, device)
    key = (gx, gy, order, tuple(tile) if order == "tile" else (1, 1), num_clusters, device)
    p = _plans.get(key)
    if p is None:
        p = cc.Plan(gx, gy, order, num_clusters, tile=tile, device=device)
        _plans[key] = p
    return p


def _dev(t: torch.Tensor) -> int:
    if not t.is_cuda:
        raise cc.CtaclustError(-1, "libctaclust operates on CUDA tensors only")
    return t.device.index or 0


def _launch(kernel, args, backend, order, tile, num_clusters, device, stream, user_order=None, **kw):
    p = plan_for(kernel, args, order, tile, num_clusters, device, user_order)
    return cc.launch(p, kernel, args, cc.make_opts(backend, **kw), stream)


def matvec(A, x, y=None, backend="agent", order=None, tile=None, num_clusters=0, stream=None, **kw):
    """y (+)= A x  (Listing 2).  y is accumulated into when given, else zero-initialised."""
    y = torch.zeros(A.shape[0], dtype=torch.float32, device=A.device) if y is None else y
    _launch("matvec", cc.matvec_args(A, x, y), backend, order, tile, num_clusters, _dev(A), stream, **kw)
    return y


def atax(A, x, backend="agent", order=None, tile=None, num_clusters=0, stream=None, out=None, **kw):
    tmp, y = out if out is not None else (torch.empty(A.shape[0], device=A.device), torch.empty(A.shape[1], device=A.device))
    _launch("atax", cc.atax_args(A, x, tmp, y), backend, order, tile, num_clusters, _dev(A), stream, **kw)
    return tmp, y


def atax_fused(A, x, backend="agent", order=None, tile=None, num_clusters=0, stream=None, out=None, **kw):
    """One-pass ATAX (CC_K_ATAX_FUSED): tmp = A x, y = A^T tmp over one read of A
    (persistent backends; n <= 16384)."""
    tmp, y = out if out is not None else (torch.empty(A.shape[0], device=A.device), torch.empty(A.shape[1], device=A.device))
    _launch("atax_fused", cc.atax_args(A, x, tmp, y), backend, order, tile, num_clusters, _dev(A), stream, **kw)
    return tmp, y


def bicg(A, p, r, backend="agent", order=None, tile=None, num_clusters=0, stream=None, out=None, **kw):
    q, s = out if out is not None else (torch.empty(A.shape[0], device=A.device), torch.empty(A.shape[1], device=A.device))
    _launch("bicg", cc.bicg_args(A, p, r, q, s), backend, order, tile, num_clusters, _dev(A), stream, **kw)
    return q, s


def mvt(A, y1, y2, x1, x2, backend="agent", order=None, tile=None, num_clusters=0, stream=None, **kw):
    """In place: x1 += A y1 ; x2 += A^T y2."""
    _launch("mvt", cc.mvt_args(A, y1, y2, x1, x2), backend, order, tile, num_clusters, _dev(A), stream, **kw)
    return x1, x2


def jacobi5(a, b, iters, backend="agent", order=None, tile=None, num_clusters=0, stream=None, row_window=None,
            fuse=1, **kw):
    """`iters` sweeps ping-ponging a <-> b; returns the buffer holding the result.
    `row_window` = (lo, hi) writes only output rows [lo, hi) of each sweep;
    `fuse` = sweeps per launch (1-4, bit-identical)."""
    args, flag = cc.jacobi5_args(a, b, iters, row_window=row_window, fuse=fuse)
    _launch("jacobi5", args, backend, order, tile, num_clusters, _dev(a), stream, **kw)
    return b if flag.value else a


def jacobi5_wave(a, b, iters, fuse=4, backend="agent", order=None, tile=None, num_clusters=0, stream=None,
                 tile_rows=0, **kw):
    """`iters` sweeps, `fuse` (1-8) per launch, by warp agents streaming column
    strips (CC_K_JACOBI5_WAVE, reading R34); COL clusters let an agent carry
    its sweep levels from one tile to the one below.  Bit-identical to
    jacobi5; returns the buffer holding the result."""
    args, flag = cc.jacobi5_args(a, b, iters, fuse=fuse, tile_rows=tile_rows)
    _launch("jacobi5_wave", args, backend, order, tile, num_clusters, _dev(a), stream, **kw)
    return b if flag.value else a


def jacobi5_halo(a, b, iters, sweep0=0, ll=None, up_ll=None, dn_ll=None, status=None, backend="agent", order=None,
                 tile=None, num_clusters=0, stream=None, **kw):
    """One slab's sweeps sweep0+1 .. sweep0+iters with the halo exchange fused
    into the sweep kernel (CC_K_JACOBI5_HALO, S§8(f)4).  `ll`: this slab's LL
    buffer (int64, cc.ll_words(cols) words); `up_ll` / `dn_ll`: the neighbours'
    LL buffers as addresses valid here, or None.  Returns the buffer holding
    this slab's result."""
    args, flag = cc.jacobi5_halo_args(a, b, iters, sweep0, ll, up_ll, dn_ll, status)
    _launch("jacobi5_halo", args, backend, order, tile, num_clusters, _dev(a), stream, **kw)
    return b if flag.value else a


def _like(t):
    """an output with t's shape and strides (the C ABI has one leading dimension for in and out)"""
    return torch.empty_strided(t.shape, t.stride(), dtype=t.dtype, device=t.device)


def conv2d(inp, w, out=None, backend="agent", order=None, tile=None, num_clusters=0, stream=None, **kw):
    out = _like(inp) if out is None else out
    args, _w = cc.conv2d_args(inp, out, w)
    _launch("conv2d", args, backend, order, tile, num_clusters, _dev(inp), stream, **kw)
    return out


class SpmvMatrix:
    """A CSR matrix resident on the device plus its merge-path split table.

    hot = H > 0 runs the inspector (cc_spmv_inspect) once: the H most
    referenced columns become hub slots, `col_kernel` holds the encoded
    column array and every launch gathers the hub values into a dense array
    read through L1 (the hub-column form of cc_spmv_args)."""

    def __init__(self, row_ptr, col, val, n_cols=None, stream=None, hot: int = 0):
        self.row_ptr, self.col, self.val = row_ptr, col, val
        self.rows = row_ptr.numel() - 1
        self.cols = self.rows if n_cols is None else n_cols
        dev = row_ptr.device
        x = torch.empty(0, device=dev)
        probe = cc.SpmvArgs(self.rows, self.cols, col.numel(), row_ptr.data_ptr(), col.data_ptr(),
                            val.data_ptr(), x.data_ptr(), x.data_ptr(), None)
        gx, _ = cc.kernel_grid("spmv", probe)
        self.part = torch.empty(gx + 1, dtype=torch.int32, device=dev)
        cc.spmv_partition(probe, self.part, stream)
        self.col_kernel, self.hot, self.xh, self.n_hot = col, None, None, 0
        if hot > 0:
            self.hot = torch.empty(hot, dtype=torch.int32, device=dev)
            self.col_kernel = torch.empty_like(col)
            scratch = torch.empty(self.cols + 65536 + 2, dtype=torch.int32, device=dev)
            self.n_hot = cc.spmv_inspect(probe, hot, self.hot, self.col_kernel, scratch, stream)
            self.xh = torch.empty(max(self.n_hot, 1), dtype=torch.float32, device=dev)

    def args(self, x, y) -> cc.SpmvArgs:
        return cc.SpmvArgs(self.rows, self.cols, self.col.numel(), self.row_ptr.data_ptr(),
                           self.col_kernel.data_ptr(), self.val.data_ptr(), x.data_ptr(), y.data_ptr(),
                           self.part.data_ptr(), None if self.hot is None else self.hot.data_ptr(),
                           None if self.xh is None else self.xh.data_ptr(), self.n_hot)


def spmv(Amat: SpmvMatrix, x, y=None, backend="agent", order=None, tile=None, num_clusters=0, stream=None,
         shub=False, **kw):
    """y = A x.  shub=True: the hottest cc.SPMV_SHUB_SLOTS hub values in each
    agent's shared memory (CC_K_SPMV_SHUB, persistent backends)."""
    y = torch.empty(Amat.rows, dtype=torch.float32, device=x.device) if y is None else y
    _launch("spmv_shub" if shub else "spmv", Amat.args(x, y), backend, order, tile, num_clusters, _dev(x), stream,
            **kw)
    return y


def hist64(data, counts=None, backend="agent", order=None, tile=None, num_clusters=0, stream=None, **kw):
    """64-bin histogram of a uint8 device tensor (bin = byte >> 2, reading R24);
    returns uint32[64] counts (zeroed by the call)."""
    if data.dtype != torch.uint8 or not data.is_contiguous():
        raise cc.CtaclustError(-1, "hist64 expects a contiguous uint8 tensor")
    counts = torch.empty(64, dtype=torch.int32, device=data.device) if counts is None else counts
    _launch("hist64", cc.hist64_args(data, counts), backend, order, tile, num_clusters, _dev(data), stream, **kw)
    return counts


def census(gx, gy, backend="agent", order="row", tile=(1, 1), num_clusters=0, device=0, stream=None,
           user_order=None, with_map=True, **kw):
    """Run the empty body over a gx x gy grid; returns (census, exec_sm, map, plan)."""
    args = cc.CensusArgs(gx, gy)
    p = plan_for("census", args, order, tile, num_clusters, device, user_order)
    dv = torch.device("cuda", device)
    cen = torch.zeros(gx * gy, dtype=torch.int32, device=dv)
    sm = torch.full((gx * gy,), -1, dtype=torch.int32, device=dv)
    mp = torch.full((gx * gy,), -1, dtype=torch.int32, device=dv) if with_map else None
    cc.launch(p, "census", args, cc.make_opts(backend, census=cen, exec_sm=sm, map=mp, **kw), stream)
    return cen, sm, mp, p
