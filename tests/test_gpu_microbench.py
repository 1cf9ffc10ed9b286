"""GPU: the Listing 3 microbenchmark runs on sm_100a and shows what section 3.1
claims for L1: the first CTA on an SM misses, CTAs dispatched to the same SM
later find the line in L1 (temporal inter-CTA locality)."""
import pytest

from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, microbench as mb

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("stagger", [0, 1200])
def test_listing3(stagger):
    info = cc.device_info()
    smid, ticks = mb.run(turnarounds=2, stagger=stagger)
    assert len(smid) == info["num_sms"] * mb.SLOTS * 2
    assert smid.min() >= 0 and smid.max() < info["smid_span"]
    r = mb.analyze(smid, ticks, num_sms=info["num_sms"])
    assert r["sms_used"] == info["num_sms"]
    assert (ticks > 0).all()
    assert r["ticks_later_turnarounds_median"] < r["ticks_first_cta_per_sm_median"]
