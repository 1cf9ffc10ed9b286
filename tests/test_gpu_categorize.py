"""GPU: the Fig. 11 categorizer end to end (timing probes -> verdict ->
tuned configuration), and the configuration it picks still matches the oracle."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_asplos_lis0l0c17_b200 import categorize as C, ctaclust as cc, ops, synth

pytestmark = pytest.mark.gpu


def _relerr(got, ref):
    return float(np.max(np.abs(np.asarray(got, np.float64) - ref) / np.maximum(np.abs(ref), 1e-30)))


def test_categorize_and_tune_bicg():
    m, n = 1000, 2312
    A = synth.matrix(3, m, n, backend="torch", device="cuda")
    p = synth.uniform(11, n, backend="torch", device="cuda")
    r = synth.uniform(12, m, backend="torch", device="cuda")
    run = lambda **kw: ops.bicg(A, p, r, **kw)
    sig = C.probe_timing(run, reps=5, has_l1_staging=False)
    assert all(x.time_ms > 0 for x in (sig.default, sig.rd_x, sig.rd_y))
    v = C.categorize(sig)
    assert v.category in C.CATEGORIES
    cands = C.candidates(v, cc.max_agents("bicg"), has_staging=False)
    tr = C.tune(run, cands, reps=3)
    assert tr.best_ms <= tr.default_ms and tr.best in [n_ for n_, _ in cands]
    q, s = ops.bicg(A, p, r, **tr.best_kw)
    torch.cuda.synchronize()
    rq, rs = O.bicg(A.cpu().numpy(), p.cpu().numpy(), r.cpu().numpy())
    assert _relerr(q.cpu().numpy(), rq) <= 1e-4 and _relerr(s.cpu().numpy(), rs) <= 1e-4


def test_categorize_and_tune_conv_with_l1_probe():
    N, R = 600, 1
    img = synth.matrix(5, N, N, backend="torch", device="cuda")
    w = synth.uniform(6, 9).reshape(3, 3).astype(np.float32)
    out = torch.zeros_like(img)
    run = lambda **kw: ops.conv2d(img, w, out=out, **kw)
    sig = C.probe_timing(run, reps=5, has_l1_staging=True)
    assert sig.l1_on.time_ms > 0 and sig.l1_off.time_ms > 0
    v = C.categorize(sig)
    tr = C.tune(run, C.candidates(v, cc.max_agents("conv2d"), has_staging=True), reps=3)
    out.zero_()
    ops.conv2d(img, w, out=out, **tr.best_kw)
    torch.cuda.synchronize()
    ref = O.conv2d(img.cpu().numpy(), w)
    got = out.cpu().numpy()
    assert _relerr(got[R:N - R, R:N - R], ref[R:N - R, R:N - R]) <= 1e-4
