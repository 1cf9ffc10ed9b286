"""Host logic of the section 4.4 / Fig. 11 categorizer (categorize.py): the
decision tree on signals shaped like the paper's description of each category
(P:2275-2277), the ncu CSV reader, candidate sets and the tuner's choice."""
import os
import sys

import pytest

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_lis0l0c17_b200 import categorize as C  # noqa: E402

P = C.Probe


def sig(d, x, y, on=None, off=None, w=False):
    return C.Signals(default=d, rd_x=x, rd_y=y, l1_on=on, l1_off=off, writes_shifted_reads=w)


def test_algorithm_related_rd_moves_l1_hit_rate():
    # an imposed order moves the L1 hit rate; L1 on/off does not change L2 -> algorithm
    s = sig(P(1.0, 10.0, 1000), P(1.0, 11.0, 990), P(0.9, 30.0, 800), on=P(l2_sectors=800), off=P(l2_sectors=805))
    v = C.categorize(s)
    assert (v.category, v.partition, v.potential) == ("algorithm", "row", True)
    assert v.optimizations == ["CLU", "TOT", "BPS"]


def test_cache_line_related_l1_off_cuts_l2():
    s = sig(P(1.0, 5.0, 1000), P(0.8, 12.0, 700), P(1.0, 5.0, 1000), on=P(l2_sectors=1000), off=P(l2_sectors=600))
    v = C.categorize(s)
    assert (v.category, v.partition) == ("cache-line", "col")


def test_partition_prefers_fewer_l2_sectors_then_time():
    base = P(1.0, 5.0, 1000)
    # significantly fewer sectors decide even when the other order is faster
    v = C.categorize(sig(base, P(0.95, 5.0, 850), P(0.80, 5.0, 950)))
    assert v.partition == "col"
    # a sector difference below the threshold is a tie: time decides
    v = C.categorize(sig(base, P(0.95, 5.0, 900), P(0.80, 5.0, 901)))
    assert v.partition == "row"
    # no sector counts: the faster order
    v = C.categorize(sig(P(1.0), P(1.2), P(0.9)))
    assert v.partition == "row" and v.potential


def test_streaming_and_data_related_by_coalescing_degree():
    flat = lambda eff: sig(P(1.0, 5.0, 1000, eff), P(1.01, 5.5, 1010), P(0.99, 4.8, 995))
    v = C.categorize(flat(100.0))
    assert (v.category, v.potential, v.partition) == ("streaming", False, None)
    assert v.optimizations == ["PFH", "TOT"]
    assert C.categorize(flat(12.5)).category == "data"
    assert C.categorize(flat(None)).category == "streaming"


def test_writing_related_from_static_analysis():
    s = sig(P(1.0, 5.0, 1000, 100.0), P(1.0, 5.0, 1000), P(1.0, 5.0, 1000), w=True)
    assert C.categorize(s).category == "writing"


def test_thresholds_are_strict_about_significance():
    th = C.Thresholds()
    just_below = sig(P(1.0, 10.0, 1000, 90.0), P(1.0 + 0.99 * th.time_rel, 10.0 + 0.99 * th.l1_hit_pp,
                                                  1000 * (1 + 0.99 * th.l2_rel)), P(1.0, 10.0, 1000))
    assert not C.categorize(just_below).potential
    at = sig(P(1.0, 10.0, 1000, 90.0), P(1.0, 10.0 + th.l1_hit_pp, 1000), P(1.0, 10.0, 1000))
    assert C.categorize(at).potential


def test_candidates_cover_tot_sweep_and_bps():
    v = C.Verdict("cache-line", "col", True, ["CLU", "TOT", "BPS"])
    names = [n for n, _ in C.candidates(v, 4)]
    assert names[0] == "default"
    assert [n for n in names if "TOT" in n] == [f"CLU-col+TOT{a}" for a in range(1, 5)]
    assert ("CLU-row", dict(backend="agent", order="row")) in C.candidates(v, 4)
    assert ("PFH-identity", dict(backend="identity")) in C.candidates(v, 4)
    assert "CLU-col+L1" in names and "CLU-col+direct" in names
    assert all(kw.get("order", "col") == "col" for n, kw in C.candidates(v, 4) if n not in ("CLU-row", "PFH-identity"))
    assert not any("L1" in n for n, _ in C.candidates(v, 4, has_staging=False))
    nv = C.Verdict("data", None, False, ["PFH", "TOT"])
    names = [n for n, _ in C.candidates(nv, 3)]
    assert names[:5] == ["default", "PFH-row-s1", "PFH-row-s2", "PFH-row-s4", "PFH-identity"]
    assert names[5:] == [f"PFH-row+TOT{a}" for a in range(1, 4)]


def test_tune_picks_fastest_with_fake_timer():
    cost = {"default": 3.0, "CLU-row+TOT1": 5.0, "CLU-row+TOT2": 2.0, "CLU-row+TOT3": 2.5}
    cands = [(n, dict(tag=n)) for n in cost]
    seen = []
    r = C.tune(lambda **kw: seen.append(kw["tag"]), cands, reps=1,
               timer=lambda fn, reps: (fn(), cost[seen[-1]])[1])
    assert (r.best, r.best_ms, r.default_ms) == ("CLU-row+TOT2", 2.0, 3.0)
    assert r.best_kw == {"tag": "CLU-row+TOT2"} and r.speedup == 1.5
    assert [n for n, _ in r.table] == list(cost)


def test_probe_from_ncu_csv(tmp_path):
    hdr = ('"ID","Process ID","Process Name","Host Name","Kernel Name","Context","Stream","Block Size",'
           '"Grid Size","Device","CC","Section Name","Metric Name","Metric Unit","Metric Value"')
    rows = []
    for i, (t, hit, sec, eff) in enumerate([(1000, 10.0, 100, 50.0), (3000, 30.0, 300, 100.0)]):
        for m, u, v in [("gpu__time_duration.sum", "nsecond", t), ("l1tex__t_sector_hit_rate.pct", "%", hit),
                        ("lts__t_sectors_srcunit_tex.sum", "sector", f"{sec:,}"),
                        ("smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct", "%", eff)]:
            rows.append(f'"{i}","1","python","h","void k(Sched)","1","7","(256, 1, 1)","(9, 1, 1)","0","10.0",'
                        f'"Command line profiler metrics","{m}","{u}","{v}"')
    f = tmp_path / "m.csv"
    f.write_text("==PROF== Connected\n" + hdr + "\n" + "\n".join(rows) + "\n")
    p = C.probe_from_ncu_csv(str(f))
    assert p.time_ms == pytest.approx(0.004)
    assert p.l2_sectors == 400
    assert p.l1_hit_pct == pytest.approx((10 * 1000 + 30 * 3000) / 4000)      # time-weighted
    assert p.ld_efficiency_pct == pytest.approx((50 * 1000 + 100 * 3000) / 4000)
    with pytest.raises(ValueError):
        (tmp_path / "e.csv").write_text("nothing\n")
        C.probe_from_ncu_csv(str(tmp_path / "e.csv"))
