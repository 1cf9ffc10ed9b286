"""Host logic of the config-3 driver with the wavefront kernel (no GPU):
JacobiSlab.calls() splits `iters` sweeps into library calls of K fused
sweeps -- iters // K full launches, then one launch of the remainder."""
import pytest

from paper_conf_asplos_lis0l0c17_b200 import drivers


def slab(iters, fuse, kname="jacobi5_wave"):
    d = drivers.JacobiSlab.__new__(drivers.JacobiSlab)
    d.iters, d.fuse, d.kname = iters, fuse, kname
    d.x = drivers.Exchange()
    return d


@pytest.mark.parametrize("iters", [1, 2, 3, 7, 8, 9, 13, 16, 17, 99, 100, 101])
@pytest.mark.parametrize("fuse", [1, 2, 3, 4, 5, 6, 7, 8])
def test_calls_cover_iters_with_bounded_fuse(iters, fuse):
    d = slab(iters, fuse)
    calls = d.calls()
    assert sum(it for it, _ in calls) == iters
    assert all(1 <= k <= fuse and it % k == 0 for it, k in calls)
    full, r = divmod(iters, fuse)
    assert d.launches_per_step() == sum(it // k for it, k in calls) == full + (1 if r else 0)


def test_bench_schedule():
    assert slab(100, 8).calls() == [(96, 8), (4, 4)]          # 12 + 1 launches (odd: two graphs)
    assert slab(100, 8).launches_per_step() == 13
    assert slab(100, 5).calls() == [(100, 5)]


def test_tile_fused_kernel_unchanged():
    assert slab(100, 3, "jacobi5").calls() == [(100, 3)]
