"""Per-rank drivers of the BASELINE configs, sharded over G GPUs.

One process per GPU.  Each driver owns this rank's shard of one config's
inputs on the device and runs one "step" of the hot path on it -- the
library's kernels through ``ops`` plus the config's exchange step through an
:class:`Exchange` -- asynchronously on the current stream.  The data-path
exchanges are exactly the ones S§8(e) lists:

* ATAX / BICG / MVT (config 2): rows of A per rank; the three transposed
  products are summed over the ranks with ONE all-reduce per step.
* Jacobi (config 3): slabs of rows + one halo row per side; per sweep the
  boundary tile rows are computed first, then the halo exchange runs on a
  communication stream while the interior tile rows compute (the classic
  boundary-first overlap); the whole 100-sweep step can be captured in one
  CUDA graph.
* conv2d (config 4): slabs + R halo rows; one exchange per step.
* SpMV (config 5): nnz-balanced row blocks (merge-path measure), x replicated,
  y all-gathered (padded blocks).

At world = 1 every driver is the unsharded computation with no exchange.
Nothing here does arithmetic of the method: kernels run in libctaclust,
exchanges in NCCL (the library's communicator) or, for the multi-process
tests on one GPU, torch.distributed.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import ctaclust as cc
from . import ops, shard, synth


# ----------------------------------------------------------------------------
# exchanges
# ----------------------------------------------------------------------------
class Exchange:
    """The collective steps a driver needs.  world == 1: all no-ops."""
    world, rank = 1, 0

    def allreduce_sum(self, t, stream=None):
        pass

    def halo_exchange(self, slab, halo, stream=None):
        pass

    def allgather(self, send, recv, stream=None):
        recv[: send.numel()].copy_(send)

    @property
    def capturable(self) -> bool:
        return True


class LibExchange(Exchange):
    """NCCL through the library's own communicator (cc_comm_*, cc_halo_exchange,
    cc_allreduce_sum, cc_allgather); rank 0's unique id travels over the
    torch.distributed process group.  Capturable into CUDA graphs."""

    def __init__(self, world: int, rank: int, device: int):
        self.world, self.rank = world, rank
        box = [cc.Comm.unique_id() if rank == 0 else None]
        if world > 1:
            dist.broadcast_object_list(box, src=0)
        self.comm = cc.Comm(box[0], world, rank, device)

    def allreduce_sum(self, t, stream=None):
        self.comm.allreduce_sum(t, stream)

    def halo_exchange(self, slab, halo, stream=None):
        self.comm.halo_exchange(slab, halo, stream)

    def allgather(self, send, recv, stream=None):
        self.comm.allgather(send, recv, stream)


class TorchExchange(Exchange):
    """torch.distributed collectives; device tensors are staged through host
    memory when the backend is gloo (several ranks sharing one GPU in the
    multi-process GPU tests, where NCCL refuses duplicate devices).  Not
    capturable."""

    def __init__(self):
        self.world, self.rank = dist.get_world_size(), dist.get_rank()
        self.staged = dist.get_backend() == "gloo"

    @property
    def capturable(self) -> bool:
        return False

    def _h(self, t):
        return t.cpu() if self.staged and t.is_cuda else t

    def allreduce_sum(self, t, stream=None):
        if self.world == 1:
            return
        h = self._h(t)
        dist.all_reduce(h, op=dist.ReduceOp.SUM)
        if h is not t:
            t.copy_(h)

    def halo_exchange(self, slab, halo, stream=None):
        if self.world == 1 or halo == 0:
            return
        up, dn = self.rank > 0, self.rank < self.world - 1
        rows = slab.shape[0]
        own0, own1 = (halo if up else 0), (rows - halo if dn else rows)
        reqs, bufs = [], {}
        if up:
            reqs.append(dist.isend(self._h(slab[own0: own0 + halo].contiguous()), self.rank - 1))
            bufs["top"] = self._h(torch.empty_like(slab[0:halo]))
            reqs.append(dist.irecv(bufs["top"], self.rank - 1))
        if dn:
            reqs.append(dist.isend(self._h(slab[own1 - halo: own1].contiguous()), self.rank + 1))
            bufs["bot"] = self._h(torch.empty_like(slab[0:halo]))
            reqs.append(dist.irecv(bufs["bot"], self.rank + 1))
        for r in reqs:
            r.wait()
        if up:
            slab[0:halo].copy_(bufs["top"])
        if dn:
            slab[rows - halo: rows].copy_(bufs["bot"])

    def allgather(self, send, recv, stream=None):
        if self.world == 1:
            recv[: send.numel()].copy_(send)
            return
        out = [self._h(torch.empty_like(send)) for _ in range(self.world)]
        dist.all_gather(out, self._h(send.contiguous()))
        recv.copy_(torch.cat([o.to(recv.device) for o in out]))


def make_exchange(kind: str, world: int, rank: int, device: int) -> Exchange:
    if world == 1:
        return Exchange()
    if kind == "nccl":
        return LibExchange(world, rank, device)
    return TorchExchange()


# ----------------------------------------------------------------------------
# config 2: ATAX + BICG + MVT, row-sharded
# ----------------------------------------------------------------------------
def atax_family_bytes(m: int, n: int) -> dict:
    """Algorithmic bytes of one ATAX + BICG + MVT step over an m x n A: the
    minimum each needs -- A read once (ATAX too: the one-pass schedule,
    CC_K_ATAX_FUSED, shows one read suffices; round 1 counted the two-pass
    form's two reads), vectors read once, outputs written once, MVT's x1 / x2
    read and written."""
    A = 4 * m * n
    atax = A + 4 * n + 4 * m + 4 * n
    bicg = A + 4 * (n + m) + 4 * (m + n)
    mvt = A + 4 * (n + m) + 8 * (m + n)
    return {"atax": atax, "bicg": bicg, "mvt": mvt, "total": atax + bicg + mvt}


class AtaxFamily:
    """Rank `rank`'s rows [lo, hi) of the n x n problem (seeds as DESIGN §4).

    State: x1 (row-indexed, local) and x2 (column-indexed, replicated) carry
    over steps (MVT accumulates in place).  The column-indexed outputs y, s, x2
    share one buffer so one all-reduce per step sums them.  Every step the
    ranks other than 0 zero their x2 slice before MVT, so after the sum
    x2 = x2_prev + sum over ranks of A_g^T y2_g (rank 0 carries x2_prev)."""

    def __init__(self, n: int, xchg: Exchange, device, m_total: int | None = None, fused_atax: bool = True):
        self.n, self.x = n, xchg
        # ATAX as one pass (CC_K_ATAX_FUSED) on the persistent backends; the
        # one-shot backends (default / redirect) keep the two-pass kernels,
        # since a one-shot CTA per row would flush y once per row
        self.fused_atax = fused_atax and n <= 16384
        self.m_total = n if m_total is None else m_total
        self.lo, self.hi = shard.row_range(self.m_total, xchg.world, xchg.rank)
        m = self.m = self.hi - self.lo
        dev = self.dev = torch.device(device)
        self.A = synth.matrix(3, m, n, backend="torch", device=dev, row0=self.lo)
        col = lambda seed: synth.uniform(seed, n, backend="torch", device=dev)
        row = lambda seed: synth.uniform(seed, m, self.lo, backend="torch", device=dev)
        self.xv, self.p, self.y1 = col(10), col(11), col(15)
        self.r, self.x1_0, self.y2 = row(12), row(13), row(16)
        self.x2_0 = col(14)
        self.tsum = torch.empty(3 * n, device=dev)
        self.y, self.s, self.x2 = self.tsum[:n], self.tsum[n:2 * n], self.tsum[2 * n:]
        self.tmp, self.q = torch.empty(m, device=dev), torch.empty(m, device=dev)
        self.x1 = torch.empty(m, device=dev)
        self.reset()

    def reset(self):
        """Back to the initial state (x1 = x1_0, x2 = x2_0)."""
        self.x1.copy_(self.x1_0)
        self.x2.copy_(self.x2_0)

    def inputs(self) -> dict:
        return dict(A=self.A, x=self.xv, p=self.p, r=self.r, y1=self.y1, y2=self.y2, x1=self.x1, x2=self.x2)

    def outputs(self) -> dict:
        return dict(tmp=self.tmp, y=self.y, q=self.q, s=self.s, x1=self.x1, x2=self.x2)

    def step(self, opts: dict, stream=None, ev=None) -> int:
        """One ATAX + BICG + MVT step (+ the all-reduce at world > 1).  `ev`:
        optional 4 events recorded around the three kernels.  Returns the
        number of library kernels queued."""
        nl = 0
        if ev is not None:
            ev[0].record(stream)
        fused = self.fused_atax and opts.get("backend", "agent") in ("agent", "identity", "static")
        if fused:
            o = dict(opts)
            o.pop("order", None)                       # one row per logical CTA: row clusters
            o.pop("staging", None)
            nl += _launch("atax_fused", cc.atax_args(self.A, self.xv, self.tmp, self.y), dict(o, order="row"), stream)
        else:
            nl += _launch("atax", cc.atax_args(self.A, self.xv, self.tmp, self.y), opts, stream)
        if ev is not None:
            ev[1].record(stream)
        nl += _launch("bicg", cc.bicg_args(self.A, self.p, self.r, self.q, self.s), opts, stream)
        if ev is not None:
            ev[2].record(stream)
        if self.x.world > 1 and self.x.rank != 0:
            self.x2.zero_()
        nl += _launch("mvt", cc.mvt_args(self.A, self.y1, self.y2, self.x1, self.x2), opts, stream)
        if ev is not None:
            ev[3].record(stream)
        self.x.allreduce_sum(self.tsum, stream)
        return nl

    def bytes_per_step(self) -> int:
        return atax_family_bytes(self.m_total, self.n)["total"]


def _launch(kernel, args, opts, stream, **plan_kw):
    kw = dict(opts)
    order = kw.pop("order", None)
    tile = kw.pop("tile", None)
    num_clusters = kw.pop("num_clusters", 0)
    dev = torch.cuda.current_device()
    p = ops.plan_for(kernel, args, order, tile, num_clusters, dev, **plan_kw)
    return cc.launch(p, kernel, args, cc.make_opts(**kw), stream)


# ----------------------------------------------------------------------------
# config 3: Jacobi, slab-sharded with boundary-first overlap
# ----------------------------------------------------------------------------
def sweep_windows(own0: int, own1: int, band: int = 32):
    """Row windows of one overlapped sweep of a slab whose owned local rows are
    [own0, own1) (own1 - own0 > 2 * band): the two boundary windows -- the
    first and last `band` owned rows, computed first because the halo
    exchange sends their edge rows -- and the interior window between them
    (None when empty).  Together they cover the owned rows exactly once."""
    t1, b0 = own0 + band, own1 - band
    assert b0 >= t1, "slab too thin to split"
    return [(own0, t1), (b0, own1)], ((t1, b0) if b0 > t1 else None)


class JacobiSlab:
    """This rank's slab of the rows x cols Jacobi (u0 = seed 4), `iters` sweeps
    per step.

    Per sweep (world > 1, overlap on): the first and last owned tile rows are
    computed first (row windows of CC_K_JACOBI5); the halo exchange of the
    freshly written boundary rows runs on `comm_stream` while the interior
    rows compute; the next sweep waits for both.  Without overlap (or at
    world = 1) a sweep is one launch, then the exchange.

    halo="fused" (world > 1): no exchange step at all -- each sweep is one
    CC_K_JACOBI5_HALO launch that stores its boundary rows as {value, sweep}
    words straight into the neighbours' LL buffers (peer memory mapped with
    CUDA IPC, shard.PeerHaloSlab) and reads its own (S§8(f)4).  Sweeps are
    numbered absolutely across steps (the LL tags), so fused steps run
    eagerly (a replayed graph would repeat the tags)."""

    def __init__(self, rows: int, cols: int, iters: int, xchg: Exchange, device, overlap: bool = True,
                 halo: str = "exchange", fuse: int = 1, kernel: str = "tile", tile_rows: int = 0):
        self.rows, self.cols, self.iters, self.x = rows, cols, iters, xchg
        # kernel="wave": the K fused sweeps run as strip wavefronts
        # (CC_K_JACOBI5_WAVE, R34, K <= 8); "tile": tile-fused (CC_K_JACOBI5, K <= 4)
        self.kname = "jacobi5_wave" if kernel == "wave" and halo != "fused" else "jacobi5"
        self.trows = tile_rows                                     # wave: logical CTA height (0 = 64)
        # K sweeps per launch (R32).  Sharded, the slab keeps K halo rows per
        # side and exchanges them once per K sweeps: a slab edge acts as a fixed
        # boundary inside the launch, so after K sweeps the error it causes has
        # reached halo row K-1 at most and every owned row is exact.
        self.fuse = fuse if halo != "fused" else 1
        self.hw = self.fuse if xchg.world > 1 else 1               # halo rows per side
        self.lo, self.hi, self.llo, self.lhi = shard.slab_range(rows, xchg.world, xchg.rank, self.hw)
        L = self.lhi - self.llo
        dev = self.dev = torch.device(device)
        ld = (cols + 3) & ~3
        self.u0 = synth.matrix(4, L, cols, backend="torch", device=dev, row0=self.llo, ld=ld)[:, :cols]
        self.a = torch.zeros(L, ld, device=dev)[:, :cols]
        self.b = torch.zeros(L, ld, device=dev)[:, :cols]
        own0, own1 = self.lo - self.llo, self.hi - self.llo
        self.own = (own0, own1)
        self.overlap = overlap and xchg.world > 1 and own1 - own0 > 64 and self.fuse == 1
        if self.overlap:
            self.windows_b, self.window_i = sweep_windows(own0, own1)
        self.comm_stream = torch.cuda.Stream(device=dev) if xchg.world > 1 else None
        self.ev_b = [torch.cuda.Event() for _ in range(2)]
        self.ev_x = [torch.cuda.Event() for _ in range(2)]
        self.graph, self.gi = None, 0
        self.fused = halo == "fused" and xchg.world > 1
        self.peer = None
        if self.fused:
            self.overlap = False
            self.a.copy_(self.u0)
            self.peer = shard.PeerHaloSlab(self.a, self.b, xchg.world, xchg.rank)
        self.sweep = 0
        self.reset()

    def reset(self):
        self.a.copy_(self.u0)
        self.b.copy_(self.u0)        # boundary rows / halo rows defined in both buffers
        if self.fused:               # restart at sweep 1: every rank's LL buffer zero first
            self.peer.ll.zero_()
            self.peer.status.zero_()
            torch.cuda.synchronize(self.dev)
            if self.x.world > 1:
                dist.barrier()
        self.sweep = 0

    def _sweep_fused(self, src, dst, opts, stream):
        pr = self.peer
        args, _ = cc.jacobi5_halo_args(src, dst, 1, self.sweep, pr.ll, pr.up_ll, pr.dn_ll, pr.status)
        self.sweep += 1
        return _launch("jacobi5_halo", args, opts, stream)

    def _sweep(self, src, dst, opts, stream, k):
        nl = 0
        if self.fused:
            return self._sweep_fused(src, dst, opts, stream)
        if not self.overlap:
            nl += _launch("jacobi5", cc.jacobi5_args(src, dst, 1)[0], opts, stream)
            self.x.halo_exchange(dst, 1, stream)
            return nl
        cur = torch.cuda.current_stream() if stream is None else stream
        for w in self.windows_b:
            nl += _launch("jacobi5", cc.jacobi5_args(src, dst, 1, row_window=w)[0], opts, stream)
        eb, ex = self.ev_b[k & 1], self.ev_x[k & 1]
        eb.record(cur)
        self.comm_stream.wait_event(eb)
        with torch.cuda.stream(self.comm_stream):
            self.x.halo_exchange(dst, 1, self.comm_stream)
        ex.record(self.comm_stream)
        if self.window_i is not None:
            nl += _launch("jacobi5", cc.jacobi5_args(src, dst, 1, row_window=self.window_i)[0], opts, stream)
        cur.wait_event(ex)
        return nl

    def step(self, opts: dict, stream=None) -> int:
        """`iters` sweeps; the result is in self.result() afterwards.  The
        buffers ping-pong within the step and the step starts from a (an even
        `iters` returns the result to a; odd steps alternate)."""
        if self.graph is not None:
            g, n = self.graph[self.gi]
            g.replay()
            if len(self.graph) == 2:                   # odd launch count: the step ended in the other buffer
                self.a, self.b = self.b, self.a
                self.gi ^= 1
            return n
        if (self.fuse > 1 or self.kname == "jacobi5_wave") and self.x.world == 1:
            nl = 0
            for it, k in self.calls():
                args, flag = cc.jacobi5_args(self.a, self.b, it, fuse=k, tile_rows=self.trows)
                nl += _launch(self.kname, args, opts, stream)
                if flag.value:
                    self.a, self.b = self.b, self.a
            return nl
        if self.fuse > 1:                                 # sharded: K sweeps, then the K-row halo exchange
            nl, done = 0, 0
            while done < self.iters:
                k = min(self.fuse, self.iters - done)
                args, flag = cc.jacobi5_args(self.a, self.b, k, fuse=k if k > 1 else 1, tile_rows=self.trows)
                nl += _launch(self.kname, args, opts, stream)
                if flag.value:
                    self.a, self.b = self.b, self.a
                self.x.halo_exchange(self.a, self.hw, stream)
                done += k
            return nl
        nl = 0
        for k in range(self.iters):
            src, dst = (self.a, self.b) if k % 2 == 0 else (self.b, self.a)
            nl += self._sweep(src, dst, opts, stream, k)
        if self.iters % 2:
            self.a, self.b = self.b, self.a
        return nl

    def calls(self):
        """(iters, fuse) per library call of an unsharded step: the iters // K
        full launches, then one launch of the remaining iters % K sweeps."""
        K = max(1, self.fuse)
        full, r = divmod(self.iters, K)
        if self.kname == "jacobi5" and K > 1:       # CC_K_JACOBI5 runs the remainder one sweep per launch
            return [(self.iters, K)]
        return ([(full * K, K)] if full else []) + ([(r, r)] if r else [])

    def launches_per_step(self) -> int:
        if self.kname == "jacobi5_wave" and self.x.world == 1:
            return sum(-(-it // k) for it, k in self.calls())
        if self.fuse > 1 and self.x.world == 1:
            return self.iters // self.fuse + self.iters % self.fuse
        if self.fuse > 1:
            return -(-self.iters // self.fuse)
        return self.iters

    def capture(self, opts: dict) -> bool:
        """Capture one step (all `iters` sweeps, both streams) into a CUDA graph;
        later steps replay it.  A step with an odd number of ping-pong launches
        ends in the other buffer, so it is captured twice, once from each
        buffer, and the replays alternate.  Plans and tensor maps are created
        by an eager step first (no allocation is legal during capture).
        Returns False when the exchange cannot be captured."""
        if not self.x.capturable or self.fused:
            return False
        self.graph = None
        self.step(opts)
        torch.cuda.synchronize()
        graphs = []
        s = torch.cuda.Stream(device=self.dev)
        s.wait_stream(torch.cuda.current_stream())
        for _ in range(2 if self.launches_per_step() % 2 else 1):
            g = torch.cuda.CUDAGraph()
            with torch.cuda.stream(s):
                with torch.cuda.graph(g, stream=s):
                    n = self.step(opts)            # records; the host-side buffer swap follows the recorded step
            graphs.append((g, n))
        torch.cuda.current_stream().wait_stream(s)
        self.graph, self.gi = graphs, 0           # graphs[gi] starts from the current self.a
        return True

    def result(self):
        """Owned rows of the field after the last step."""
        return self.a[self.own[0]: self.own[1]]

    def bytes_per_step(self) -> int:
        """one read and one write of the field per launch: per sweep unfused,
        per K sweeps with K fused sweeps per launch (R32)"""
        return 8 * self.rows * self.cols * self.launches_per_step()


class GraphStep:
    """Mixin: capture one step (all its launches and exchanges) into a CUDA
    graph and replay it -- removes the host-side marshalling of each call from
    the timed region.  The first (eager) step creates the plans and tensor
    maps; nothing is allocated during capture."""
    graph = None

    def capture(self, opts: dict) -> bool:
        if not self.x.capturable:
            return False
        self.graph = None
        self.step(opts)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        s = torch.cuda.Stream(device=self.dev)
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            with torch.cuda.graph(g, stream=s):
                n = self.step(opts)
        torch.cuda.current_stream().wait_stream(s)
        self.graph, self.graph_launches = g, n
        return True

    def step(self, opts: dict, stream=None) -> int:
        if self.graph is not None:
            self.graph.replay()
            return self.graph_launches
        return self.step_eager(opts, stream)


# ----------------------------------------------------------------------------
# config 4: conv2d, slab-sharded
# ----------------------------------------------------------------------------
class ConvSlab(GraphStep):
    """This rank's slab (owned rows + R halo rows per side) of the rows x cols
    image (seed 5), filter seed 6 normalised to sum 1.  One step =
    the halo exchange (world > 1) + one conv launch; owned output rows are
    exact (every owned row is >= R rows from a slab edge that is not the
    image border)."""

    def __init__(self, rows: int, cols: int, R: int, xchg: Exchange, device, w=None):
        self.rows, self.cols, self.R, self.x = rows, cols, R, xchg
        self.lo, self.hi, self.llo, self.lhi = shard.slab_range(rows, xchg.world, xchg.rank, R)
        dev = self.dev = torch.device(device)
        K = 2 * R + 1
        if w is None:
            import numpy as np
            w = synth.uniform(6, K * K).reshape(K, K)
            w = (w / w.astype(np.float64).sum()).astype(np.float32)
        self.w = w
        ld = (cols + 3) & ~3                       # 16-byte rows (TMA strides, float4 access)
        self.inp = synth.matrix(5, self.lhi - self.llo, cols, ld=ld, backend="torch", device=dev,
                                row0=self.llo)[:, :cols]
        self.out = torch.empty(self.lhi - self.llo, ld, device=dev)[:, :cols]

    def inputs(self) -> dict:
        return dict(inp=self.inp)

    def outputs(self) -> dict:
        return dict(out=self.result())

    def step_eager(self, opts: dict, stream=None) -> int:
        self.x.halo_exchange(self.inp, self.R, stream)
        args, self._w = cc.conv2d_args(self.inp, self.out, self.w)
        return _launch("conv2d", args, opts, stream)

    def result(self):
        return self.out[self.lo - self.llo: self.hi - self.llo]

    def bytes_per_step(self) -> int:
        return 8 * self.rows * self.cols

    def flops_per_step(self) -> int:
        return 2 * (2 * self.R + 1) ** 2 * (self.rows - 2 * self.R) * (self.cols - 2 * self.R)


# ----------------------------------------------------------------------------
# config 5: CSR SpMV, nnz-balanced row blocks
# ----------------------------------------------------------------------------
class SpmvBlock(GraphStep):
    """This rank's nnz-balanced row block of the R-MAT matrix (seed 7, values
    seed 8, x seed 9).  x is replicated; one step = local SpMV + all-gather of
    y (blocks padded to the largest)."""

    def __init__(self, scale: int, xchg: Exchange, device, edge_factor: int = 16, hot: int = 0):
        self.x = xchg
        dev = self.dev = torch.device(device)
        rp, col = synth.rmat_csr(7, scale, edge_factor, backend="torch", device=dev)
        self.rows, self.nnz = rp.numel() - 1, col.numel()
        val = synth.uniform(8, self.nnz, backend="torch", device=dev)
        self.xv = synth.uniform(9, self.rows, backend="torch", device=dev)
        self.lo, self.hi = shard.spmv_row_range(rp, xchg.world, xchg.rank)
        if xchg.world > 1:
            lrp, lcol, lval = shard.spmv_local(rp, col, val, self.lo, self.hi)
            lrp, lcol, lval = lrp.contiguous(), lcol.contiguous(), lval.contiguous()
            del rp, col, val
        else:
            lrp, lcol, lval = rp, col, val
        self.A = ops.SpmvMatrix(lrp, lcol, lval, n_cols=self.rows, hot=hot)
        self.local_nnz = lcol.numel()
        self.cap = self._cap(xchg)
        self.y = torch.zeros(self.cap, device=dev)
        self.yall = torch.zeros(self.cap * xchg.world, device=dev)

    def _cap(self, xchg):
        """rows of the largest block (the padded all-gather's block size)"""
        if xchg.world == 1:
            return self.hi - self.lo
        n = torch.tensor([self.hi - self.lo], device=self.dev if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(n, op=dist.ReduceOp.MAX)
        return int(n.item())

    def step_eager(self, opts: dict, stream=None) -> int:
        nl = _launch_spmv(self.A, self.xv, self.y, opts, stream)
        if self.x.world > 1:
            self.x.allgather(self.y, self.yall, stream)
        return nl

    def bytes_per_step(self) -> int:
        return 8 * self.nnz + 4 * (self.rows + 1) + 8 * self.rows


def _launch_spmv(Am, x, y, opts, stream):
    kw = dict(opts)
    shub = kw.pop("shub", False)              # CC_K_SPMV_SHUB: hub tier in the agents' shared memory
    return _launch("spmv_shub" if shub else "spmv", Am.args(x, y), kw, stream)
