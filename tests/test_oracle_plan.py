"""Pins for the schedule oracle (oracle/plan.py) against what the paper fixes.

The oracle builds the partition by sorting CTAs by their indexing key and
cutting balanced chunks.  The checks below come from elsewhere: the paper's
worked examples (tests/golden/worked_examples.json), its closed forms (Eq. 7,
Listing 4, Listing 5 PARAM_CALL/_jobs/_base, the Fig. 7 indexing formulas)
and brute-force invariants.  A dropped "+1", a swapped (bx, by), a wrong
chunk boundary or a transposed tile order fails at least one of them.
"""
import json
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import plan as P

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "worked_examples.json")))


# --- worked examples printed in the paper --------------------------------
def test_partition_worked_example():
    g = GOLD["partition_example"]
    v = g["cta_by"] * g["gx"] + g["cta_bx"]          # row-major indexing
    assert v == g["v"]
    assert P.f(g["gx"] * g["gy"], g["M"], v) == (g["w"], g["i"])


@pytest.mark.parametrize("key", ["invert_example", "invert_example_fig8c"])
def test_invert_worked_examples(key):
    g = GOLD[key]
    assert P.f_inv(g["V"], g["M"], g["w"], g["i"]) == g["v"]


def test_rr_binding_worked_example():
    g = GOLD["rr_binding_example"]
    assert P.rd_binding(g["u"], g["M"]) == (g["w"], g["i"])


def test_fig8_clusters():
    g = GOLD["fig8_clusters"]
    pl = P.plan(g["gx"], g["gy"], P.ROW, g["M"])
    off = pl["offsets"]
    got = [list(pl["perm"][off[i]:off[i + 1]]) for i in range(g["M"])]
    assert got == g["clusters"]


# --- closed forms from the paper -------------------------------------------
def eq7(V, M, w, i):
    """Eq. 7: v = i*(|V|/M + 1) + w + min(|V|%M - i, 0)."""
    return i * (V // M + 1) + w + min(V % M - i, 0)


def listing5_jobs_base(V, M, sm):
    """Listing 5 l.14-15 with PARAM_CALL l.32-33 under reading R3 (_cn = ctas/SM + 1)."""
    cd, ck, cn = V // M, V % M, V // M + 1
    jobs = cd + (1 if sm < ck else 0)
    base = cn * sm + ((ck - sm) if (ck - sm) < 0 else 0)
    return jobs, base


@pytest.mark.parametrize("V", range(0, 80))
def test_eq7_and_listing5_match_oracle_partition(V):
    for M in range(1, V + 4):
        sizes = P.cluster_sizes(V, M)
        start = 0
        for i in range(M):
            jobs, base = listing5_jobs_base(V, M, i)
            assert jobs == sizes[i]
            if sizes[i]:
                assert base == start
            for w in range(sizes[i]):
                v = P.f_inv(V, M, w, i)
                assert v == eq7(V, M, w, i) == start + w
                assert P.f(V, M, v) == (w, i)
            start += sizes[i]
        assert start == V


def test_printed_eq4_condition_is_not_the_inverse_of_eq7():
    """Documents reading R1: the printed 'if v%M <= |V|%M' branch of Eq. 4/5
    disagrees with Eq. 7 (first failure |V|=5, M=4, v=4); the reading
    'v < r(q+1)' agrees everywhere."""
    V, M, v = 5, 4, 4
    q, r = divmod(V, M)
    printed = (v % (q + 1), v // (q + 1)) if v % M <= r else (v % q, (v - r) // q)
    assert eq7(V, M, *printed) != v
    reading = (v % (q + 1), v // (q + 1)) if v < r * (q + 1) else ((v - r) % q, (v - r) // q)
    assert eq7(V, M, *reading) == v == P.f_inv(V, M, *P.f(V, M, v))


@pytest.mark.parametrize("V", range(1, 80))
def test_listing4_redirection_is_a_bijection(V):
    for M in range(1, V + 3):
        vs = sorted(P.rd_redirect(V, M, u) for u in range(V))
        assert vs == list(range(V))


def test_listing4_fig8c_redirect_order():
    # 3x2 grid on 2 SMs: u -> (w,i) = (u/2, u%2) -> v; Fig. 8(C) SM0 serves v 0,1,2
    V, M = 6, 2
    order = [P.rd_redirect(V, M, u) for u in range(V)]
    assert order == [0, 3, 1, 4, 2, 5]
    assert sorted(order[0::2]) == GOLD["fig8_clusters"]["clusters"][0]


# --- indexing methods (Fig. 7) ---------------------------------------------
@pytest.mark.parametrize("gx,gy", [(1, 1), (3, 2), (5, 7), (12, 1), (1, 9), (8, 8)])
def test_row_and_col_indexing_formulas(gx, gy):
    seq_r = P.order_sequence(gx, gy, P.ROW)
    seq_c = P.order_sequence(gx, gy, P.COL)
    for by in range(gy):
        for bx in range(gx):
            lin = by * gx + bx
            assert seq_r[by * gx + bx] == lin
            assert seq_c[bx * gy + by] == lin


def tile_v(gx, gy, tw, th, bx, by):
    """Reading R6 closed form for the clipped tile-wise order."""
    tX, tY = bx // tw, by // th
    w_t = min(tw, gx - tX * tw)
    h_t = min(th, gy - tY * th)
    return tY * th * gx + h_t * tX * tw + (by - tY * th) * w_t + (bx - tX * tw)


@pytest.mark.parametrize("gx,gy,tw,th", [(4, 4, 2, 2), (5, 7, 2, 3), (12, 12, 4, 4),
                                         (7, 3, 8, 8), (9, 10, 3, 1), (1, 6, 1, 4)])
def test_tile_indexing_formula(gx, gy, tw, th):
    seq = P.order_sequence(gx, gy, P.TILE, tw, th)
    for by in range(gy):
        for bx in range(gx):
            assert seq[tile_v(gx, gy, tw, th, bx, by)] == by * gx + bx


def test_tile_order_small_picture():
    # 4x4 grid, 2x2 tiles: first tile is CTAs (0,0),(1,0),(0,1),(1,1) -> lin 0,1,4,5
    seq = P.order_sequence(4, 4, P.TILE, 2, 2)
    assert list(seq[:8]) == [0, 1, 4, 5, 2, 3, 6, 7]


# --- brute-force invariants on tiny grids ----------------------------------
def check_invariants(pl, gx, gy, M):
    V = gx * gy
    perm, off = pl["perm"], pl["offsets"]
    assert sorted(perm.tolist()) == list(range(V))               # every CTA exactly once
    sizes = np.diff(off)
    q, r = divmod(V, M)
    assert set(sizes.tolist()) <= {q, q + 1}
    assert all(sizes[:r] == q + 1) and all(sizes[r:] == q)       # first r larger (l.14)
    assert off[0] == 0 and off[-1] == V


@pytest.mark.parametrize("order", [P.ROW, P.COL, P.TILE])
def test_tiny_grid_brute_force(order):
    for gx in range(1, 8):
        for gy in range(1, 8):
            V = gx * gy
            for M in (1, 2, 3, 5, V, V + 2):
                pl = P.plan(gx, gy, order, M, 2, 3)
                check_invariants(pl, gx, gy, M)
                seq = P.order_sequence(gx, gy, order, 2, 3)
                # contiguity: cluster i is exactly positions off[i]..off[i+1]-1
                for i in range(M):
                    a, b = pl["offsets"][i], pl["offsets"][i + 1]
                    assert list(pl["perm"][a:b]) == list(seq[a:b])


@settings(max_examples=60, deadline=None)
@given(gx=st.integers(1, 40), gy=st.integers(1, 40), M=st.integers(1, 200),
       tw=st.integers(1, 9), th=st.integers(1, 9), seed=st.integers(0, 10))
def test_property_user_order(gx, gy, M, tw, th, seed):
    V = gx * gy
    rng = np.random.default_rng(seed)
    u = rng.permutation(V)
    pl = P.plan(gx, gy, P.USER, M, user_order=u)
    check_invariants(pl, gx, gy, M)
    assert np.array_equal(pl["perm"], u)
    pl2 = P.plan(gx, gy, P.TILE, M, tw, th)
    check_invariants(pl2, gx, gy, M)


def test_user_order_rejects_non_permutation():
    with pytest.raises(ValueError):
        P.plan(2, 2, P.USER, 2, user_order=[0, 1, 1, 3])


def test_config_grids_q_r():
    # SURVEY §8(a) a2 (q, r) for M = 148 at the BASELINE configs
    for V, qr in [(1024, (6, 136)), (32768, (221, 60)), (4096, (27, 100)),
                  (262144, (1771, 36)), (65536, (442, 120))]:
        pl = P.plan(V, 1, P.ROW, 148)
        assert (pl["q"], pl["r"]) == qr
