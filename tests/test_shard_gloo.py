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
