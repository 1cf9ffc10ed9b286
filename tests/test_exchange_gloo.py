"""CPU multi-process (gloo, world 2 and 3) check of the drivers' exchange layer
(drivers.TorchExchange): the halo exchange of slab decompositions (halo 1 and
3, the Jacobi and conv 7x7 cases), the all-reduce and the padded all-gather.
The GPU drivers call the same methods (or the library's NCCL equivalents with
the same contract, include/ctaclust.h cc_halo_exchange)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_lis0l0c17_b200 import shard


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    from paper_conf_asplos_lis0l0c17_b200 import drivers
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    X = drivers.make_exchange("torch", world, rank, 0)
    res = {}
    rows, cols = 23, 7
    glob = torch.arange(rows * cols, dtype=torch.float32).reshape(rows, cols)
    for halo in (1, 3):
        lo, hi, llo, lhi = shard.slab_range(rows, world, rank, halo)
        slab = glob[llo:lhi].clone()
        own0, own1 = lo - llo, hi - llo
        slab[:own0] = -1                      # stale halo rows
        slab[own1:] = -1
        X.halo_exchange(slab, halo)
        res[f"halo{halo}"] = bool(torch.equal(slab, glob[llo:lhi]))
    t = torch.full((5,), float(rank + 1))
    X.allreduce_sum(t)
    res["allreduce"] = bool(torch.all(t == world * (world + 1) / 2))
    send = torch.full((4,), float(rank))
    recv = torch.empty(4 * world)
    X.allgather(send, recv)
    res["allgather"] = bool(torch.equal(recv, torch.arange(world).float().repeat_interleave(4)))
    q.put((rank, res))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_torch_exchange(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    for r in range(world):
        assert all(out[r].values()), (r, out[r])


def test_world1_exchange_is_noop():
    from paper_conf_asplos_lis0l0c17_b200 import drivers
    X = drivers.make_exchange("nccl", 1, 0, 0)
    t = torch.ones(3)
    X.allreduce_sum(t)
    X.halo_exchange(t.view(3, 1), 1)
    assert torch.equal(t, torch.ones(3))
    r = torch.zeros(3)
    X.allgather(t, r)
    assert torch.equal(r, t)


def test_sweep_windows_cover_owned_rows_once():
    from paper_conf_asplos_lis0l0c17_b200 import drivers
    for rows, world in ((16384, 8), (330, 2), (330, 4), (1000, 3)):
        for g in range(world):
            lo, hi, llo, lhi = shard.slab_range(rows, world, g, 1)
            own0, own1 = lo - llo, hi - llo
            if own1 - own0 <= 64:
                continue
            wb, wi = drivers.sweep_windows(own0, own1)
            cover = np.zeros(lhi - llo, np.int64)
            for a, b in wb + ([wi] if wi else []):
                cover[a:b] += 1
            assert np.all(cover[own0:own1] == 1)            # every owned row exactly once
            assert not cover[:own0].any() and not cover[own1:].any()   # halo rows never written
            assert wb[0][0] == own0 and wb[1][1] == own1        # the exchanged edge rows are in the boundary windows
