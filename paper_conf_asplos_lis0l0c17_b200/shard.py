"""Row sharding of the ATAX/BICG/MVT family over G GPUs.

Rank g owns rows [row_lo(g), row_hi(g)) of A and the matching slices of the
row-indexed vectors; column-indexed inputs are replicated.  The row products
(A x, A p, A y1) are then purely local; the transposed products (A^T tmp,
A^T r, A^T y2) are sums over all row blocks, so each rank produces a partial
n-vector and one all-reduce (NCCL over NVLink; gloo in the CPU tests) forms
the total -- the only data-path exchange.  ATAX needs no exchange between its
passes: pass 2 consumes exactly the tmp rows pass 1 produced locally.
Row-indexed outputs are gathered at the end (all-gather).

`compute` callables do the per-rank arithmetic (the CUDA kernels in bench and
users' code; the oracle in the CPU tests); this module only moves vectors.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def row_range(n_rows: int, world: int, rank: int) -> tuple[int, int]:
    """Balanced contiguous row blocks: the first n_rows % world ranks get one more."""
    q, r = divmod(n_rows, world)
    lo = rank * q + min(rank, r)
    return lo, lo + q + (1 if rank < r else 0)


def _allreduce(t: torch.Tensor, world: int):
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return t


def _allgather_rows(local: torch.Tensor, n_rows: int, world: int) -> torch.Tensor:
    if world == 1:
        return local
    sizes = [row_range(n_rows, world, g) for g in range(world)]
    cap = max(hi - lo for lo, hi in sizes)
    buf = torch.zeros(cap, dtype=local.dtype, device=local.device)
    buf[: local.numel()] = local
    out = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(out, buf)
    return torch.cat([out[g][: hi - lo] for g, (lo, hi) in enumerate(sizes)])


def sharded_step(compute, n_rows: int, world: int, rank: int, gather: bool = True) -> dict:
    """One ATAX + BICG + MVT step on this rank's row block.

    ``compute(lo, hi)`` runs the local kernels and returns a dict with the
    row-part outputs ``tmp``, ``q``, ``x1`` (length hi-lo) and the partial
    column-part outputs ``y``, ``s``, ``x2d`` (length n; x2d is the A^T y2
    contribution only).  Returns the combined results (x2 = x2_init + sum x2d
    is left to the caller, which owns x2_init)."""
    lo, hi = row_range(n_rows, world, rank)
    part = compute(lo, hi)
    for key in ("y", "s", "x2d"):
        _allreduce(part[key], world)
    if gather:
        for key in ("tmp", "q", "x1"):
            part[key] = _allgather_rows(part[key], n_rows, world)
    return part


# --------------------------------------------------------------------------
# Slab sharding of the stencils (Jacobi, conv2d): rank g owns image rows
# [lo, hi) and keeps H halo rows on each side that are not global boundary.
# One halo exchange per Jacobi sweep (point-to-point with the two neighbours:
# NCCL send/recv over NVLink on GPUs, gloo in the CPU tests); conv2d needs one
# exchange before its single pass.  The per-slab sweep treats the slab's first
# and last rows as fixed boundary -- exactly what a halo row is during a sweep.
# --------------------------------------------------------------------------
def slab_range(rows: int, world: int, rank: int, halo: int = 1) -> tuple[int, int, int, int]:
    """(lo, hi, llo, lhi): owned rows [lo, hi) and local rows [llo, lhi)."""
    lo, hi = row_range(rows, world, rank)
    return lo, hi, max(lo - halo, 0), min(hi + halo, rows)


def exchange_halos(buf: torch.Tensor, rows: int, world: int, rank: int, halo: int = 1):
    """Refresh the halo rows of the local slab `buf` (local rows [llo, lhi)) with
    the neighbours' owned boundary rows."""
    if world == 1:
        return
    lo, hi, llo, lhi = slab_range(rows, world, rank, halo)
    reqs = []
    if rank > 0:         # my first owned rows -> rank-1 ; its last owned rows -> my top halo
        reqs.append(dist.isend(buf[lo - llo: lo - llo + halo].contiguous(), rank - 1))
        top = torch.empty_like(buf[0:halo])
        reqs.append(dist.irecv(top, rank - 1))
    if rank < world - 1:  # my last owned rows -> rank+1 ; its first owned rows -> my bottom halo
        reqs.append(dist.isend(buf[hi - halo - llo: hi - llo].contiguous(), rank + 1))
        bot = torch.empty_like(buf[0:halo])
        reqs.append(dist.irecv(bot, rank + 1))
    for r in reqs:
        r.wait()
    if rank > 0:
        buf[0:halo] = top
    if rank < world - 1:
        buf[lhi - llo - halo: lhi - llo] = bot


def jacobi_slab(sweep, a: torch.Tensor, b: torch.Tensor, iters: int, rows: int, world: int, rank: int):
    """`iters` sweeps of the sharded Jacobi.  `sweep(src, dst)` runs one sweep on
    the local slab (global boundary and halo rows copied through).  Returns the
    local buffer holding the result."""
    src, dst = a, b
    for _ in range(iters):
        sweep(src, dst)
        exchange_halos(dst, rows, world, rank, 1)
        src, dst = dst, src
    return src


def conv_slab(conv, slab: torch.Tensor, rows: int, world: int, rank: int, R: int) -> torch.Tensor:
    """Slab-sharded 2D convolution (S§8(e)): one exchange of the R halo rows on
    each side, then `conv(slab)` on the local slab (its edges act as image
    borders: every owned row is at least R rows from an edge that is not the
    global border, so the owned outputs equal the unsharded ones).  Returns the
    owned rows of the output."""
    exchange_halos(slab, rows, world, rank, R)
    lo, hi, llo, _ = slab_range(rows, world, rank, R)
    return conv(slab)[lo - llo: hi - llo]


def spmv_row_range(row_ptr, world: int, rank: int) -> tuple[int, int]:
    """nnz-balanced contiguous rows for CSR SpMV (S§8(e)): rank g owns rows
    [lo, hi) with lo the first row whose start is >= g * (rows + nnz) / world on
    the merged rows+nnz axis (the merge-path measure the kernel balances, so
    power-law hubs and empty rows both count)."""
    import numpy as np
    rp = np.asarray(row_ptr.cpu() if hasattr(row_ptr, "cpu") else row_ptr, dtype=np.int64)
    rows = rp.size - 1
    cost = rp[:rows] + np.arange(rows)             # merged coordinate of each row's start
    total = rows + int(rp[-1])

    def cut(g):
        if g <= 0:
            return 0
        if g >= world:
            return rows
        return int(np.searchsorted(cost, (g * total) // world, side="left"))
    return cut(rank), cut(rank + 1)


def spmv_local(row_ptr, col, val, lo: int, hi: int):
    """The CSR block of rows [lo, hi): (row_ptr rebased to 0, col, val) views."""
    base = int(row_ptr[lo])
    end = int(row_ptr[hi])
    return row_ptr[lo: hi + 1] - base, col[base:end], val[base:end]


def gather_rows(local_owned: torch.Tensor, rows: int, world: int, rank: int) -> torch.Tensor:
    """All-gather the owned row blocks of a 2D slab decomposition (final gather)."""
    if world == 1:
        return local_owned
    cap = max(hi - lo for lo, hi in (row_range(rows, world, g) for g in range(world)))
    buf = torch.zeros((cap,) + tuple(local_owned.shape[1:]), dtype=local_owned.dtype, device=local_owned.device)
    buf[: local_owned.shape[0]] = local_owned
    out = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(out, buf)
    return torch.cat([out[g][: row_range(rows, world, g)[1] - row_range(rows, world, g)[0]] for g in range(world)])


# --------------------------------------------------------------------------
# Fused peer-memory halo (S§8(f)4, CC_K_JACOBI5_HALO): instead of a separate
# exchange per sweep, each rank's sweep kernel stores its boundary rows, each
# value tagged with the sweep number, straight into the neighbours' LL buffers
# (NVLink peer mappings opened with CUDA IPC); the neighbour's next sweep polls
# the tags.  The host only wires the neighbours once; no collective per sweep.
# --------------------------------------------------------------------------
def neighbours(world: int, rank: int) -> tuple[int | None, int | None]:
    """(upper, lower) neighbour ranks of a slab decomposition, None at the ends."""
    return (rank - 1 if rank > 0 else None), (rank + 1 if rank < world - 1 else None)


class PeerHaloSlab:
    """This rank's slab buffers a/b (owned rows plus halo rows, as slab_range),
    its LL buffer, and the mapped addresses of its neighbours' LL buffers.

    Collective over the process group at construction (one all_gather_object
    of IPC handles) and at `close`; `sweeps` runs with no host exchange."""

    def __init__(self, a: torch.Tensor, b: torch.Tensor, world: int, rank: int):
        from . import ctaclust as cc
        self.cc, self.a, self.b, self.world, self.rank = cc, a, b, world, rank
        self.device = a.device.index or 0
        self.ll = torch.zeros(cc.ll_words(a.shape[1]), dtype=torch.int64, device=a.device)
        self.status = torch.zeros(1, dtype=torch.int32, device=a.device)
        mine = {"pid": __import__("os").getpid(), "ll": self.ll.data_ptr(),
                "h": cc.ipc_handle(self.ll) if world > 1 else None}
        allv = [mine]
        if world > 1:
            allv = [None] * world
            dist.all_gather_object(allv, mine)
        self._opened = []
        self.up_ll = self.dn_ll = None
        up, dn = neighbours(world, rank)
        for which, g in (("up_ll", up), ("dn_ll", dn)):
            if g is None:
                continue
            other = allv[g]
            if other["pid"] == mine["pid"]:            # same process: the address is valid as it is
                ptr = other["ll"]
            else:
                h, off = other["h"]
                base = cc.ipc_open(h, self.device)
                self._opened.append(base)
                ptr = base + off
            setattr(self, which, ptr)
        torch.cuda.synchronize(self.device)
        if world > 1:
            dist.barrier()                             # every rank's LL buffer is zero before any sweep

    def sweeps(self, iters: int, sweep0: int = 0, **kw) -> torch.Tensor:
        from . import ops
        return ops.jacobi5_halo(self.a, self.b, iters, sweep0, self.ll, self.up_ll, self.dn_ll, self.status, **kw)

    def close(self):
        torch.cuda.synchronize(self.device)
        if self.world > 1:
            dist.barrier()                             # no neighbour still stores into our buffer
        for base in self._opened:
            self.cc.ipc_close(base)
        self._opened = []
