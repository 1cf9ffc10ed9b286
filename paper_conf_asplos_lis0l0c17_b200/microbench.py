"""The paper's Listing 3 microbenchmark (section 3.1) on B200:
launch it through the C ABI (`cc_l1_reuse_probe`) and reduce its per-CTA
(smid, cycles) record to the paper's three observations:

(1) temporal inter-CTA locality -- in default order only the first
    turnaround of CTAs on an SM pays the miss; later CTAs on that SM hit the
    line in L1 (Fig. 2(A));
(2) spatial inter-CTA locality -- with staggered starts only the first CTA
    of the first turnaround misses (Fig. 2(B));
(3) the hardware CTA dispatch pattern: which SMs the first wave
    covers and how consecutive CTA ids spread over SMs.

The kernel (csrc/k_microbench.cuh) does the measuring; this module only
launches it and summarises host-side.
"""
from __future__ import annotations

import numpy as np

from . import ctaclust as cc

SLOTS = 32           # resident one-warp CTAs per SM on sm_100a (hardware CTA limit)


def run(turnarounds: int = 2, stagger: int = 0, device: int = 0, ctas: int | None = None):
    """Launch Listing 3 with `num_sms * SLOTS * turnarounds` CTAs (l.18-22) and
    return (smid, ticks) as numpy arrays."""
    import torch
    info = cc.device_info(device)
    n = ctas if ctas is not None else info["num_sms"] * SLOTS * turnarounds
    dev = torch.device("cuda", device)
    inp = torch.ones(32 * info["smid_span"], dtype=torch.float32, device=dev)
    smid = torch.full((n,), -1, dtype=torch.int32, device=dev)
    ticks = torch.zeros(n, dtype=torch.int32, device=dev)
    sink = torch.zeros(n, dtype=torch.float32, device=dev)
    cc.l1_reuse_probe(n, stagger, inp, smid, ticks, sink)
    torch.cuda.synchronize(dev)
    return smid.cpu().numpy(), ticks.cpu().numpy().view(np.uint32).astype(np.int64)


def analyze(smid: np.ndarray, ticks: np.ndarray, slots: int = SLOTS, num_sms: int | None = None) -> dict:
    """Summaries of one run (CTA ids stand for dispatch order within an SM)."""
    smid = np.asarray(smid)
    ticks = np.asarray(ticks, dtype=np.int64)
    sms = np.unique(smid)
    n_sm = num_sms if num_sms is not None else len(sms)
    first, turn0_rest, later = [], [], []
    for s in sms:
        b = np.nonzero(smid == s)[0]                    # CTA ids on this SM, ascending
        t = ticks[b]
        first.append(t[0])
        turn0_rest.extend(t[1:slots].tolist())
        later.extend(t[slots:].tolist())
    med = lambda v: float(np.median(v)) if len(v) else None
    counts = np.bincount(smid, minlength=int(smid.max()) + 1)[sms]
    s0 = smid[0]
    b0 = np.nonzero(smid == s0)[0]
    return {
        "ctas": int(len(smid)), "sms_used": int(len(sms)),
        "ticks_first_cta_per_sm_median": med(first),
        "ticks_rest_of_first_turnaround_median": med(turn0_rest),
        "ticks_later_turnarounds_median": med(later),
        "ctas_per_sm_min": int(counts.min()), "ctas_per_sm_max": int(counts.max()),
        "first_wave_distinct_sms": int(len(np.unique(smid[:n_sm]))),
        "first_wave_smids_head": smid[:16].tolist(),
        "consecutive_same_sm_frac": float(np.mean(smid[1:] == smid[:-1])) if len(smid) > 1 else 0.0,
        "sm_of_cta0": {"smid": int(s0), "cta_ids_head": b0[:12].tolist(), "ticks_head": ticks[b0[:12]].tolist()},
    }
