"""GPU: binding + agent runtime exactly-once coverage and bit-exact maps.

For every backend, order, throttle level and (fake) topology the execution
census must be exactly 1 for every logical CTA, and the slot -> CTA map the
device decoded must equal the oracle's partition table bit for bit."""
import numpy as np
import pytest
import torch

from oracle import plan as OP
from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def nsm():
    return cc.device_info(0)["num_sms"]


def test_device_facts_and_rank_table(nsm):
    info = cc.device_info(0)
    assert info["num_sms"] == torch.cuda.get_device_properties(0).multi_processor_count
    ranks = cc.sm_rank_table(0)
    seen = ranks[ranks >= 0]
    assert sorted(seen.tolist()) == list(range(len(seen)))      # dense
    assert len(seen) == nsm                                      # the probe saw every SM


GRIDS = [(1, 1), (37, 23), (32, 32), (64, 512), (3 * 148 + 5, 1)]


@pytest.mark.parametrize("gx,gy", GRIDS)
@pytest.mark.parametrize("order,tile", [("row", (1, 1)), ("col", (1, 1)), ("tile", (8, 8)), ("tile", (3, 5))])
def test_agent_census_and_map(gx, gy, order, tile, nsm):
    cen, sm, mp, p = ops.census(gx, gy, "agent", order, tile)
    torch.cuda.synchronize()
    assert torch.all(cen == 1), "exactly-once violated"
    ref = OP.plan(gx, gy, cc.ORDERS[order], nsm, *tile)
    assert np.array_equal(mp.cpu().numpy(), ref["perm"])
    assert torch.all(sm >= 0)


@pytest.mark.parametrize("gx,gy", GRIDS)
@pytest.mark.parametrize("order,tile,M", [("row", (1, 1), 0), ("col", (1, 1), 296), ("tile", (8, 8), 1000),
                                          ("row", (1, 1), 7), ("tile", (3, 5), 100000)])
def test_static_binding_census_map_and_one_sm_per_cluster(gx, gy, order, tile, M, nsm):
    """CC_BACKEND_AGENT_STATIC: CTA i runs cluster i.  Exactly once, the map is
    the oracle's partition, and -- binding by construction -- every task of a
    cluster ran on one SM (home coherence 1, exactly)."""
    cen, sm, mp, p = ops.census(gx, gy, "static", order, tile, num_clusters=M)
    torch.cuda.synchronize()
    assert torch.all(cen == 1)
    MM = M if M else nsm
    ref = OP.plan(gx, gy, cc.ORDERS[order], MM, *tile)
    assert np.array_equal(mp.cpu().numpy(), ref["perm"])
    smv, perm, off = sm.cpu().numpy(), ref["perm"], ref["offsets"]
    for i in range(min(MM, gx * gy)):
        members = perm[off[i]:off[i + 1]]
        assert len(set(smv[members].tolist())) <= 1, i


@pytest.mark.parametrize("backend", ["default", "identity", "redirect"])
@pytest.mark.parametrize("gx,gy", GRIDS)
def test_other_backends_census(backend, gx, gy, nsm):
    cen, sm, mp, p = ops.census(gx, gy, backend, "row")
    torch.cuda.synchronize()
    assert torch.all(cen == 1)
    if backend == "identity":
        assert np.array_equal(mp.cpu().numpy(), np.arange(gx * gy))
    if backend == "redirect":   # Listing 4: slot v ran CTA perm[v]
        ref = OP.plan(gx, gy, OP.ROW, nsm)
        assert np.array_equal(mp.cpu().numpy(), ref["perm"])
        red = np.array([OP.rd_redirect(gx * gy, nsm, u) for u in range(gx * gy)])
        assert sorted(red.tolist()) == list(range(gx * gy))


@pytest.mark.parametrize("active", [1, 2, 0])
@pytest.mark.parametrize("M", [7, 148, 300, 5000])
def test_throttling_and_fake_topologies(active, M):
    """Fewer/more clusters than SMs, throttled agents: coverage still exactly once
    (clusters with no home agent are stolen)."""
    gx, gy = 128, 64
    cen, sm, mp, p = ops.census(gx, gy, "agent", "tile", (4, 4), num_clusters=M, active_agents=active)
    torch.cuda.synchronize()
    assert torch.all(cen == 1)
    ref = OP.plan(gx, gy, OP.TILE, M, 4, 4)
    assert np.array_equal(mp.cpu().numpy(), ref["perm"])


def test_forced_starvation_single_agent():
    cen, *_ = ops.census(512, 16, "agent", "row", max_agents=1, active_agents=1)
    torch.cuda.synchronize()
    assert torch.all(cen == 1)


def test_home_fraction_without_stealing(nsm):
    """steal = 0 is the paper's scheme (static binding): with every SM holding
    agents the census is still complete, and every CTA runs on its home SM."""
    gx, gy = 64, 64
    cen, sm, mp, p = ops.census(gx, gy, "agent", "row", steal=0)
    torch.cuda.synchronize()
    c = cen.cpu().numpy()
    assert c.max() <= 1
    if c.min() == 1:
        ranks = cc.sm_rank_table(0)
        perm, off = p.table()
        home = np.empty(gx * gy, dtype=np.int64)
        for i in range(p.M):
            home[perm[off[i]:off[i + 1]]] = i
        ran = ranks[sm.cpu().numpy()]
        assert np.all(ran == home)


def test_repeated_launches_reset_workspace():
    args = cc.CensusArgs(200, 100)
    p = ops.plan_for("census", args, "col")
    cen = torch.zeros(20000, dtype=torch.int32, device="cuda")
    for _ in range(25):
        cc.launch(p, "census", args, cc.make_opts("agent", census=cen, active_agents=3))
    torch.cuda.synchronize()
    assert torch.all(cen == 25)


def test_user_order():
    rng = np.random.default_rng(3)
    u = rng.permutation(50 * 30).astype(np.int32)
    cen, sm, mp, p = ops.census(50, 30, "agent", user_order=u)
    torch.cuda.synchronize()
    assert torch.all(cen == 1)
    assert np.array_equal(mp.cpu().numpy(), u)


def test_workspace_ordered_across_streams():
    """Agent launches sharing a plan's self-resetting workspace never overlap:
    a launch on another stream while the previous one is still running is
    ordered after it (no error), from two host threads too, and every logical
    CTA still runs exactly once (census) in every launch."""
    import threading
    N = 16384
    a = torch.rand(N, N, device="cuda")
    b = torch.empty_like(a)
    a2, b2 = torch.rand(N, N, device="cuda"), torch.empty_like(a)
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    ops.jacobi5(a, b, 20, backend="agent", order="row", stream=sa)       # ~7 ms of sweeps on sa
    ev = torch.cuda.Event(enable_timing=True)
    ops.jacobi5(a2, b2, 1, backend="agent", order="row", stream=sb)      # queued behind sa's sweeps
    ev.record(sb)
    done_a = torch.cuda.Event(enable_timing=True)
    done_a.record(sa)
    torch.cuda.synchronize()
    assert done_a.elapsed_time(ev) >= 0                                   # sb's launch finished after sa's
    # census launches on one plan from two host threads and two streams
    args = cc.CensusArgs(512, 512)
    p = ops.plan_for("census", args, "row")
    cens = [torch.zeros(512 * 512, dtype=torch.int32, device="cuda") for _ in range(8)]
    streams = [torch.cuda.Stream() for _ in range(2)]

    def run(t):
        for k in range(t, 8, 2):
            cc.launch(p, "census", args, cc.make_opts("agent", census=cens[k]), streams[t])
    th = [threading.Thread(target=run, args=(t,)) for t in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    torch.cuda.synchronize()
    assert all(bool(torch.all(c == 1)) for c in cens)


@pytest.mark.parametrize("stages", [3, 5, 7])
def test_ring_depth_not_multiple_of_groups(stages):
    """Regression (round 2): a ring depth that is not a multiple of the body's
    consumer groups let two groups share a slot, and on full-size launches a
    group could take the parity of a fill still in flight for the other group
    (hang / launch failure).  The launcher now rounds the depth up; a large
    two-group stencil launch with such a request must be exact."""
    from paper_conf_asplos_lis0l0c17_b200 import synth
    import oracle as O
    u0 = synth.matrix(4, 8192, 8192)
    a = torch.from_numpy(u0).cuda()
    out = ops.jacobi5(a, torch.empty_like(a), 2, backend="agent", order="row", stages=stages)
    torch.cuda.synchronize()
    ref = O.jacobi5_f32(u0, 2)
    assert np.array_equal(out.cpu().numpy(), ref)
