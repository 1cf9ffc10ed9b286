"""GPU parity of the fused peer-memory halo exchange (S§8(f)4, CC_K_JACOBI5_HALO).

The slab-sharded Jacobi (S§8(e)) with the per-sweep halo exchange done inside
the sweep kernel -- boundary rows stored straight into the neighbours' halo
rows' LL buffers as {value, sweep} words, no fences -- must equal the unsharded
fp32 oracle bit for bit (S§8(c) "Multi-GPU" pin: the G-shard result equals the
1-GPU result; virtual-slab mode on one GPU).  Virtual slabs: G slabs on one
GPU, their sweeps interleaved on one stream.  The two-process case maps the
neighbour's buffers with CUDA IPC, as ranks on different GPUs do.
"""
import os
import subprocess
import sys
import textwrap

import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, shard, synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def virtual_slabs(u0, world, iters, **kw):
    """Run `iters` fused-halo sweeps over `world` virtual slabs of u0 on one GPU;
    returns (owned rows stacked, status words)."""
    rows, cols = u0.shape
    slabs = []
    for g in range(world):
        lo, hi, llo, lhi = shard.slab_range(rows, world, g, 1)
        ld = (cols + 3) & ~3                      # 16-byte rows; ragged widths keep a padded ld
        a = torch.zeros(lhi - llo, ld, device="cuda")[:, :cols]
        a.copy_(torch.from_numpy(np.ascontiguousarray(u0[llo:lhi])))
        b = torch.zeros(lhi - llo, ld, device="cuda")[:, :cols]
        ll = torch.zeros(cc.ll_words(cols), dtype=torch.int64, device="cuda")
        status = torch.zeros(1, dtype=torch.int32, device="cuda")
        slabs.append(dict(a=a, b=b, ll=ll, status=status, lo=lo, hi=hi, llo=llo))

    def nb(g):
        return slabs[g]["ll"].data_ptr() if 0 <= g < world else None

    for s in range(iters):                    # sweep s+1 of every slab, in slab order
        for g, x in enumerate(slabs):
            src, dst = (x["a"], x["b"]) if s % 2 == 0 else (x["b"], x["a"])
            ops.jacobi5_halo(src, dst, 1, s, x["ll"], nb(g - 1), nb(g + 1), x["status"], **kw)
    torch.cuda.synchronize()
    res = []
    for x in slabs:
        out = x["a"] if iters % 2 == 0 else x["b"]
        res.append(out[x["lo"] - x["llo"]: x["hi"] - x["llo"]].cpu().numpy())
    return np.concatenate(res), [int(x["status"].item()) for x in slabs]


HVARIANTS = [dict(backend="agent", order="row"), dict(backend="default"), dict(backend="identity"),
             dict(backend="agent", order="tile", tile=(2, 2), stages=2, batch=1),
             dict(backend="redirect", order="col"), dict(backend="agent", order="row", staging="direct"),
             dict(backend="default", staging="l1")]


@pytest.mark.parametrize("v", HVARIANTS, ids=lambda v: "-".join(str(x) for x in v.values()))
@pytest.mark.parametrize("world,rows,cols,iters", [(2, 150, 100, 7), (3, 97, 260, 6), (4, 130, 33, 5),
                                                    (2, 66, 64, 4)])
def test_virtual_slabs_equal_unsharded(v, world, rows, cols, iters):
    u0 = synth.matrix(4, rows, cols)
    got, status = virtual_slabs(u0, world, iters, **v)
    assert status == [0] * world
    assert np.array_equal(got, O.jacobi5_f32(u0, iters))


def test_virtual_slabs_tiny_slab_both_neighbours():
    """Slabs of 1-3 owned rows: one tile row both reads both halos and deposits
    into both neighbours."""
    u0 = synth.matrix(4, 9, 70)
    got, status = virtual_slabs(u0, 4, 5, backend="agent", order="row")
    assert status == [0] * 4
    assert np.array_equal(got, O.jacobi5_f32(u0, 5))


def test_virtual_slabs_full_width_sampled():
    """Config 3's width (16384 columns, 512 tile columns) on 8 virtual slabs,
    rows cut to 2048 so the fp32 oracle finishes: every 61st row checked."""
    rows, cols, T, G = 2048, 16384, 6, 8
    u0 = synth.matrix(4, rows, cols)
    got, status = virtual_slabs(u0, G, T, backend="agent", order="row")
    assert status == [0] * G
    ref = O.jacobi5_f32(u0, T)
    assert np.array_equal(got[::61], ref[::61])
    for g in range(1, G):                      # the rows next to every slab seam
        lo = shard.slab_range(rows, G, g, 1)[0]
        assert np.array_equal(got[lo - 2: lo + 2], ref[lo - 2: lo + 2])


@pytest.mark.parametrize("v", [dict(backend="agent", order="row", max_agents=1), dict(backend="default"),
                               dict(backend="static", order="row", num_clusters=148)],
                         ids=lambda v: v["backend"])
def test_ll_litmus_concurrent_streams(v):
    """LL protocol litmus: each virtual slab runs all its sweeps on its OWN
    stream, so neighbouring slabs' sweeps execute truly concurrently and in no
    fixed relative order (a slab may run several sweeps ahead until it blocks
    on its neighbour's tags).  Every sweep's result must still be bit-exact and
    no poll may time out: RAW (a reader takes exactly tag s-1) and WAR (a
    deposit of sweep s+2 never overwrites words of sweep s before they were
    read) under real concurrency, not only under the interleaved order."""
    rows, cols, G, T = 260, 200, 3, 24
    u0 = synth.matrix(4, rows, cols)
    slabs = []
    for g in range(G):
        lo, hi, llo, lhi = shard.slab_range(rows, G, g, 1)
        a = torch.from_numpy(np.ascontiguousarray(u0[llo:lhi])).cuda()
        slabs.append(dict(a=a, b=torch.zeros_like(a), lo=lo, hi=hi, llo=llo,
                          ll=torch.zeros(cc.ll_words(cols), dtype=torch.int64, device="cuda"),
                          status=torch.zeros(1, dtype=torch.int32, device="cuda"), st=torch.cuda.Stream()))
    torch.cuda.synchronize()

    def nb(g):
        return slabs[g]["ll"].data_ptr() if 0 <= g < G else None

    for s in range(T):                                   # queued slab by slab; streams run concurrently
        for g, x in enumerate(slabs):
            src, dst = (x["a"], x["b"]) if s % 2 == 0 else (x["b"], x["a"])
            ops.jacobi5_halo(src, dst, 1, s, x["ll"], nb(g - 1), nb(g + 1), x["status"], stream=x["st"], **v)
    torch.cuda.synchronize()
    got = np.concatenate([(x["a"] if T % 2 == 0 else x["b"])[x["lo"] - x["llo"]: x["hi"] - x["llo"]].cpu().numpy()
                          for x in slabs])
    assert [int(x["status"].item()) for x in slabs] == [0] * G
    assert np.array_equal(got, O.jacobi5_f32(u0, T))


def test_missing_neighbour_deposit_times_out_not_hangs():
    """Sweep 2 of slab 0 launched without slab 1's sweep 1: the bounded poll
    gives up after ~4 s and reports it in `status` instead of hanging."""
    u0 = synth.matrix(4, 64, 64)
    a = torch.from_numpy(u0[:33].copy()).cuda()
    b = torch.zeros_like(a)
    ll = torch.zeros(cc.ll_words(64), dtype=torch.int64, device="cuda")
    pll = torch.zeros_like(ll)
    status = torch.zeros(1, dtype=torch.int32, device="cuda")
    ops.jacobi5_halo(b, a, 1, 1, ll, None, pll.data_ptr(), status, backend="default")
    torch.cuda.synchronize()
    assert status.item() == 1


def test_argument_errors():
    a = torch.zeros(40, 64, device="cuda")
    b = torch.zeros_like(a)
    ll = torch.zeros(cc.ll_words(64), dtype=torch.int64, device="cuda")
    with pytest.raises(cc.CtaclustError) as e:          # a neighbour but no own LL buffer
        ops.jacobi5_halo(a, b, 1, 0, None, ll.data_ptr(), None)
    assert e.value.status == -1
    with pytest.raises(cc.CtaclustError) as e:          # misaligned neighbour LL
        ops.jacobi5_halo(a, b, 1, 0, ll, ll.data_ptr() + 8, None)
    assert e.value.status == -1
    with pytest.raises(cc.CtaclustError) as e:          # a 2-row slab with both halos owns nothing
        ops.jacobi5_halo(a[:2], b[:2], 1, 0, ll, ll.data_ptr(), ll.data_ptr())
    assert e.value.status == -1
    # no neighbours: the plain sweep, equal to CC_K_JACOBI5
    u0 = synth.matrix(4, 40, 64)
    x = torch.from_numpy(u0).cuda()
    out = ops.jacobi5_halo(x, torch.zeros_like(x), 3)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), O.jacobi5_f32(u0, 3))


WORKER = textwrap.dedent("""
    import os, sys, numpy as np, torch, torch.distributed as dist
    sys.path.insert(0, {root!r})
    import oracle as O
    from paper_conf_asplos_lis0l0c17_b200 import shard, synth
    rank, world = int(sys.argv[1]), int(sys.argv[2])
    dist.init_process_group("gloo", init_method="file://" + sys.argv[3], rank=rank, world_size=world)
    torch.cuda.set_device(0)
    rows, cols, T = 120, 96, 6
    u0 = synth.matrix(4, rows, cols)
    lo, hi, llo, lhi = shard.slab_range(rows, world, rank, 1)
    a = torch.from_numpy(np.ascontiguousarray(u0[llo:lhi])).cuda()
    b = torch.zeros_like(a)
    slab = shard.PeerHaloSlab(a, b, world, rank)
    out = slab.sweeps(T, backend="agent", order="row", max_agents=1)
    torch.cuda.synchronize()
    st = int(slab.status.item())
    slab.close()
    ok = st == 0 and np.array_equal(out[lo - llo: hi - llo].cpu().numpy(), O.jacobi5_f32(u0, T)[lo:hi])
    print("RESULT", rank, st, ok, flush=True)
    dist.destroy_process_group()
""")


def test_two_processes_ipc_one_gpu(tmp_path):
    """Two ranks in two processes on the same GPU: the neighbour's LL buffer is
    mapped with CUDA IPC (cc_ipc_handle / cc_ipc_open), as across GPUs.
    Without MPS the two contexts time-slice, so each sweep's wait may span a
    slice; the kernel's bounded wait keeps a failure from hanging."""
    script = tmp_path / "w.py"
    script.write_text(WORKER.format(root=ROOT))
    store = str(tmp_path / "store")            # file rendezvous: no port to race for
    procs = [subprocess.Popen([sys.executable, str(script), str(r), "2", store], stdout=subprocess.PIPE,
                              stderr=subprocess.STDOUT, text=True) for r in range(2)]
    outs = []
    for p in procs:
        try:
            outs.append(p.communicate(timeout=240)[0])
        except subprocess.TimeoutExpired:
            p.kill()
            outs.append(p.communicate()[0])
    res = [ln for o in outs for ln in o.splitlines() if ln.startswith("RESULT")]
    assert len(res) == 2, outs
    assert all(ln.endswith("True") for ln in res), outs
