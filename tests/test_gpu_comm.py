"""GPU: the NCCL exchange entry points on a one-rank communicator (the boxes of
this round have one GPU; the multi-rank exchange logic is checked with gloo in
tests/test_shard_gloo.py)."""
import pytest
import torch

from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc

pytestmark = pytest.mark.gpu


def test_single_rank_comm():
    uid = cc.Comm.unique_id()
    assert len(uid) == 128
    comm = cc.Comm(uid, 1, 0, 0)
    slab = torch.arange(40 * 33, dtype=torch.float32, device="cuda").view(40, 33)
    ref = slab.clone()
    comm.halo_exchange(slab, 1)                       # no neighbours: untouched
    v = torch.rand(1000, device="cuda")
    w = v.clone()
    comm.allreduce_sum(w)                             # sum over one rank = identity
    out = torch.empty_like(v)
    comm.allgather(v, out)
    torch.cuda.synchronize()
    assert torch.equal(slab, ref) and torch.equal(w, v) and torch.equal(out, v)
    comm.close()


def test_comm_argument_errors():
    with pytest.raises(cc.CtaclustError) as e:
        cc.Comm(b"\0" * 128, 2, 5, 0)
    assert e.value.status == -1
