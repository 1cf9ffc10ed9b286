"""Multi-process (gloo, world size 2 and 3) check of the row-sharding host logic
(shard.py): per-rank partials combined by all-reduce / all-gather must equal
the unsharded oracle result.  The per-rank arithmetic here is the CPU oracle
(test infrastructure); on GPUs it is the CUDA kernels, with the same exchange."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_lis0l0c17_b200 import shard, synth


def test_row_range_partition():
    for n in (0, 1, 7, 16384, 16385):
        for world in (1, 2, 3, 8):
            spans = [shard.row_range(n, world, g) for g in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == n
            assert all(spans[g][1] == spans[g + 1][0] for g in range(world - 1))
            sizes = [hi - lo for lo, hi in spans]
            assert max(sizes) - min(sizes) <= 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, m, n, q):
    import oracle as O
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    A = synth.matrix(3, m, n, kind="int")
    x, p = synth.small_int(10, n), synth.small_int(11, n)
    r, y1, y2, x1 = synth.small_int(12, m), synth.small_int(15, n), synth.small_int(16, m), synth.small_int(13, m)

    def compute(lo, hi):
        Ab = A[lo:hi]
        tmp, y = O.atax(Ab, x)
        qq, s = O.bicg(Ab, p, r[lo:hi])
        o1, x2d = O.mvt(Ab, x1[lo:hi], np.zeros(n, np.float32), y1, y2[lo:hi])
        t = lambda a: torch.from_numpy(np.asarray(a, dtype=np.float64))
        return {"tmp": t(tmp), "y": t(y), "q": t(qq), "s": t(s), "x1": t(o1), "x2d": t(x2d)}

    out = shard.sharded_step(compute, m, world, rank)
    if rank == 0:
        q.put({k: v.numpy() for k, v in out.items()})
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_step_equals_unsharded(world):
    import oracle as O
    m, n = 37, 29
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(g, world, port, m, n, q)) for g in range(world)]
    for pr in procs:
        pr.start()
    got = q.get(timeout=120)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    A = synth.matrix(3, m, n, kind="int")
    x, p = synth.small_int(10, n), synth.small_int(11, n)
    r, y1, y2, x1 = synth.small_int(12, m), synth.small_int(15, n), synth.small_int(16, m), synth.small_int(13, m)
    tmp, y = O.atax(A, x)
    qq, s = O.bicg(A, p, r)
    o1, o2 = O.mvt(A, x1, np.zeros(n, np.float32), y1, y2)
    # integer-exact inputs: every order of summation gives the same bits (R18)
    assert np.array_equal(got["tmp"], tmp) and np.array_equal(got["y"], y)
    assert np.array_equal(got["q"], qq) and np.array_equal(got["s"], s)
    assert np.array_equal(got["x1"], o1) and np.array_equal(got["x2d"], o2)


def _jacobi_worker(rank, world, port, R, C, T, q):
    import oracle as O
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    u0 = synth.matrix(4, R, C)
    lo, hi, llo, lhi = shard.slab_range(R, world, rank, 1)
    a = torch.from_numpy(u0[llo:lhi].copy())
    b = torch.zeros_like(a)

    def sweep(src, dst):       # one fp32 sweep of the slab (its first/last rows fixed)
        dst.copy_(torch.from_numpy(O.jacobi5_f32(src.numpy(), 1)))

    out = shard.jacobi_slab(sweep, a, b, T, R, world, rank)
    full = shard.gather_rows(out[lo - llo: hi - llo], R, world, rank)
    if rank == 0:
        q.put(full.numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_jacobi_slab_halo_exchange_is_exact(world):
    """Slab-sharded Jacobi with one halo exchange per sweep equals the unsharded
    fp32 sweep bit for bit (same evaluation order, R14)."""
    import oracle as O
    R, C, T = 23, 17, 9
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_jacobi_worker, args=(g, world, port, R, C, T, q)) for g in range(world)]
    for pr in procs:
        pr.start()
    got = q.get(timeout=120)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    assert np.array_equal(got, O.jacobi5_f32(synth.matrix(4, R, C), T))


def test_slab_range():
    for rows in (5, 16384, 17):
        for world in (1, 2, 8):
            for halo in (1, 3):
                for g in range(world):
                    lo, hi, llo, lhi = shard.slab_range(rows, world, g, halo)
                    assert 0 <= llo <= lo <= hi <= lhi <= rows
                    assert lo - llo == (halo if g > 0 and lo >= halo else lo - llo)


def _conv_worker(rank, world, port, N, M, R, q):
    import oracle as O
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    img = synth.matrix(5, N, M)
    w = synth.uniform(6, (2 * R + 1) ** 2).reshape(2 * R + 1, 2 * R + 1)
    w = (w / w.sum()).astype(np.float32)
    lo, hi, llo, lhi = shard.slab_range(N, world, rank, R)
    slab = torch.from_numpy(img[llo:lhi].copy())
    if rank > 0:                 # halo rows start stale: the exchange must fill them
        slab[: lo - llo] = -7.0
    if rank < world - 1:
        slab[hi - llo:] = -7.0
    own = shard.conv_slab(lambda t: torch.from_numpy(O.conv2d(t.numpy(), w)), slab, N, world, rank, R)
    full = shard.gather_rows(own, N, world, rank)
    if rank == 0:
        q.put((full.numpy(), w))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,R", [(2, 1), (3, 3), (3, 1)])
def test_conv_slab_equals_unsharded(world, R):
    """Slab-sharded conv with one R-row halo exchange equals the unsharded conv
    (the fp64 oracle on every slab: same terms in the same order per output)."""
    import oracle as O
    N, M = 29, 21
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_conv_worker, args=(g, world, port, N, M, R, q)) for g in range(world)]
    for pr in procs:
        pr.start()
    got, w = q.get(timeout=120)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    assert np.array_equal(got, O.conv2d(synth.matrix(5, N, M), w))


def _spmv_worker(rank, world, port, scale, q):
    import oracle as O
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    rp, col = synth.rmat_csr(7, scale, 8)
    rows = rp.size - 1
    val = synth.small_int(8, col.size)
    x = synth.small_int(9, rows)
    lo, hi = shard.spmv_row_range(rp, world, rank)
    lrp, lcol, lval = shard.spmv_local(rp, col, val, lo, hi)
    y = np.asarray(O.spmv_csr(lrp, lcol, lval, x))
    ys = [None] * world
    dist.all_gather_object(ys, (lo, hi, y))
    if rank == 0:
        q.put(ys)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_spmv_row_sharding_equals_unsharded(world):
    """nnz-balanced row blocks (x replicated): the gathered per-rank products
    equal the unsharded SpMV exactly in integer mode (R18)."""
    import oracle as O
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_spmv_worker, args=(g, world, port, 10, q)) for g in range(world)]
    for pr in procs:
        pr.start()
    parts = q.get(timeout=120)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    rp, col = synth.rmat_csr(7, 10, 8)
    val, x = synth.small_int(8, col.size), synth.small_int(9, rp.size - 1)
    ref = O.spmv_csr(rp, col, val, x)
    assert [p[0] for p in parts] == sorted(p[0] for p in parts) and parts[0][0] == 0
    assert all(parts[g][1] == parts[g + 1][0] for g in range(world - 1)) and parts[-1][1] == rp.size - 1
    assert np.array_equal(np.concatenate([p[2] for p in parts]), ref)


def test_spmv_row_range_balances_merge_cost():
    rp, col = synth.rmat_csr(7, 12, 16)
    rows, nnz = rp.size - 1, int(rp[-1])
    for world in (1, 2, 3, 8):
        spans = [shard.spmv_row_range(rp, world, g) for g in range(world)]
        assert spans[0][0] == 0 and spans[-1][1] == rows
        assert all(spans[g][1] == spans[g + 1][0] for g in range(world - 1))
        costs = [(hi - lo) + int(rp[hi] - rp[lo]) for lo, hi in spans]
        # each block within one row's cost of the even share
        max_row = int(np.max(np.diff(rp))) + 1
        assert max(costs) - (rows + nnz) / world <= max_row + 1
