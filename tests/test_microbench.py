"""Host-side reduction of the Listing 3 microbenchmark (microbench.analyze)
on synthetic records with known answers; the ABI check of cc_l1_reuse_probe."""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, microbench as mb  # noqa: E402


def test_analyze_round_robin_temporal_reuse():
    n_sm, slots, turns = 6, 4, 3
    smid = np.tile(np.arange(n_sm), slots * turns)            # pure round robin
    ticks = np.full(len(smid), 40)
    ticks[:n_sm] = 800                                        # first CTA on each SM misses
    ticks[n_sm:n_sm * slots] = 700                            # rest of turnaround 0: hit-reserved
    r = mb.analyze(smid, ticks, slots=slots)
    assert r["sms_used"] == n_sm and r["ctas"] == n_sm * slots * turns
    assert r["ticks_first_cta_per_sm_median"] == 800
    assert r["ticks_rest_of_first_turnaround_median"] == 700
    assert r["ticks_later_turnarounds_median"] == 40
    assert r["first_wave_distinct_sms"] == n_sm
    assert r["ctas_per_sm_min"] == r["ctas_per_sm_max"] == slots * turns
    assert r["consecutive_same_sm_frac"] == 0.0
    assert r["sm_of_cta0"]["cta_ids_head"][:3] == [0, n_sm, 2 * n_sm]


def test_analyze_blocked_dispatch():
    # every SM takes a block of consecutive ids (a "blocked" pattern)
    smid = np.repeat(np.array([3, 1, 2, 0]), 5)
    r = mb.analyze(smid, np.arange(20), slots=5)
    assert r["first_wave_distinct_sms"] == 1
    assert r["consecutive_same_sm_frac"] == 16 / 19
    assert r["sm_of_cta0"]["smid"] == 3 and r["sm_of_cta0"]["ticks_head"] == [0, 1, 2, 3, 4]
    assert r["ticks_later_turnarounds_median"] is None


def test_probe_abi_rejects_bad_arguments():
    L = cc.lib()
    vp = ctypes.c_void_p(1)
    assert L.cc_l1_reuse_probe(-1, 0, vp, vp, vp, vp, None) == -1
    assert L.cc_l1_reuse_probe(4, -5, vp, vp, vp, vp, None) == -1
    assert L.cc_l1_reuse_probe(4, 0, None, vp, vp, vp, None) == -1
    assert L.cc_l1_reuse_probe(0, 0, None, None, None, None, None) == 0      # no-op
