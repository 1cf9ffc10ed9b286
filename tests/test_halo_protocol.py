"""CPU model of the fused peer-halo protocol (S§8(f)4, CC_K_JACOBI5_HALO).

Host logic only, no GPU: ranks run their sweeps in stream order, the
boundary work items of a sweep in any order and any interleaving across ranks.
The rules modelled are the kernel's (k_stencil.cuh, LL form): the work item
for column group c and side d of sweep s > 1 polls its own LL buffer of parity
(s-1) & 1, side d, until the word carries tag s-1, then -- in the same thread,
data-dependent on what it read -- stores its boundary value tagged s into the
neighbour's LL buffer of parity s & 1 (the neighbour's opposite side).  A slab
with one owned row reads and deposits both sides in one item.  Checked over
random schedules: no deadlock; every read sees exactly the neighbour's
sweep-(s-1) value (RAW); no word is overwritten before the neighbour's read of
it (WAR).  A single-buffer variant must fail the WAR check.
"""
import random

import pytest

from paper_conf_asplos_lis0l0c17_b200 import shard


def run_model(world, groups, sweeps, rng, one_row=False, parities=2):
    # ll[r][parity][side][c] = tag stored (side 0 = from up, 1 = from down)
    ll = [[[[0] * groups for _ in range(2)] for _ in range(parities)] for _ in range(world)]
    # reads still owed: (r, sweep, side, c) that rank r will read at `sweep`
    sweep = [1] * world

    def items(r):
        up, dn = shard.neighbours(world, r)
        sides = [d for d, nb in ((0, up), (1, dn)) if nb is not None]
        if one_row:
            return {(c, tuple(sides)) for c in range(groups)} if sides else set()
        return {(c, (d,)) for c in range(groups) for d in sides}

    pending = [items(r) for r in range(world)]
    done = 0
    total = sum(len(p) for p in pending) * sweeps
    read_done = set()            # (r, sweep, side, c) reads completed
    while True:
        for r in range(world):   # ranks without boundary work just advance
            while sweep[r] <= sweeps and not pending[r]:
                sweep[r] += 1
                pending[r] = items(r) if sweep[r] <= sweeps else set()
        enabled = []
        for r in range(world):
            if sweep[r] > sweeps:
                continue
            s = sweep[r]
            for it in sorted(pending[r]):
                c, sides = it
                if s == 1 or all(ll[r][(s - 1) % parities][d][c] == s - 1 for d in sides):
                    enabled.append((r, it))
        if not enabled:
            break
        r, (c, sides) = rng.choice(enabled)
        s = sweep[r]
        up, dn = shard.neighbours(world, r)
        for d in sides:
            if s > 1:
                assert ll[r][(s - 1) % parities][d][c] == s - 1          # RAW: exactly sweep s-1
            read_done.add((r, s, d, c))
        for d in sides:
            nb = up if d == 0 else dn
            nd = 1 - d                               # my top row lands in the upper neighbour's bottom side
            slot = ll[nb][s % parities][nd]
            old = slot[c]
            if old >= 1:                             # WAR: its reader (sweep old+1) must be done
                assert (nb, old + 1, nd, c) in read_done, (nb, old + 1, nd, c)
            slot[c] = s
        pending[r].discard((c, sides))
        done += 1
    return done, total, sweep


@pytest.mark.parametrize("world,groups", [(2, 1), (2, 5), (3, 4), (5, 3), (8, 6)])
@pytest.mark.parametrize("one_row", [False, True])
def test_protocol_no_deadlock_exact_tags(world, groups, one_row):
    rng = random.Random(world * 100 + groups + one_row)
    sweeps = 7
    for _ in range(60):
        done, total, sweep = run_model(world, groups, sweeps, rng, one_row)
        assert done == total
        assert all(x > sweeps for x in sweep)


def test_single_parity_buffer_breaks_war():
    """With one LL buffer instead of two parities a fast neighbour's sweep s+1
    deposit overwrites the sweep-s word before it is read: the model catches it."""
    rng = random.Random(3)
    caught = 0
    for _ in range(200):
        try:
            run_model(3, 2, 5, rng, parities=1)
        except AssertionError:
            caught += 1
    assert caught > 0


def test_neighbours():
    assert shard.neighbours(1, 0) == (None, None)
    assert shard.neighbours(3, 0) == (None, 1)
    assert shard.neighbours(3, 1) == (0, 2)
    assert shard.neighbours(3, 2) == (1, None)
