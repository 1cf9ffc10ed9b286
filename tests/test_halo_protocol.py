"""CPU model of the fused peer-halo protocol (S§8(f)4, CC_K_JACOBI5_HALO).

Host logic only, no GPU: ranks run their sweeps in stream order, the boundary
tiles of a sweep in any order and any interleaving across ranks.  The rules
modelled are the kernel's (k_stencil.cuh): a boundary tile of sweep s waits
until the neighbour's flags for tile columns c-1..c+1 reach s-1, reads its halo
columns (which span tiles c-1..c+1), stores its boundary row piece into the
neighbour's destination buffer of sweep s, then raises the neighbour's flag
for column c to s.  Checked over random schedules: no deadlock, every halo
read sees exactly the neighbour's sweep s-1 data (not older: RAW; not newer:
WAR), matching what the slab decomposition needs.
"""
import random

import pytest

from paper_conf_asplos_lis0l0c17_b200 import shard


def run_model(world, gx, sweeps, rng, span=1):
    # ver[r][parity][side][c]: sweep whose boundary data sits in rank r's buffer
    # `parity`, halo side (0 top / 1 bottom), tile column c.  Sweep s reads
    # buffer (s-1)%2 and writes buffer s%2; the initial halo (sweep 0) is in 0.
    ver = [[[[0 if p == 0 else -1] * gx for _ in range(2)] for p in range(2)] for _ in range(world)]
    flags = [[[0] * gx for _ in range(2)] for _ in range(world)]   # [r][from side][c]
    sweep = [1] * world
    pending = []
    for r in range(world):
        pending.append(set(range(gx)))
    done = 0
    while True:
        enabled = []
        for r in range(world):
            if sweep[r] > sweeps:
                continue
            up, dn = shard.neighbours(world, r)
            s = sweep[r]
            for c in sorted(pending[r]):
                ok = True
                for side, nb in ((0, up), (1, dn)):
                    if nb is None:
                        continue
                    for k in range(max(c - span, 0), min(c + span, gx - 1) + 1):
                        ok &= flags[r][side][k] >= s - 1
                if ok:
                    enabled.append((r, c))
        if not enabled:
            break
        r, c = rng.choice(enabled)
        s = sweep[r]
        up, dn = shard.neighbours(world, r)
        for side, nb in ((0, up), (1, dn)):
            if nb is None:
                continue
            for k in range(max(c - 1, 0), min(c + 1, gx - 1) + 1):      # RAW and WAR in one check
                assert ver[r][(s - 1) % 2][side][k] == s - 1, (r, s, side, k)
        for side, nb in ((0, up), (1, dn)):
            if nb is None:
                continue
            nside = 1 - side                       # my top row is the upper neighbour's bottom halo
            ver[nb][s % 2][nside][c] = s
            flags[nb][nside][c] = max(flags[nb][nside][c], s)
        pending[r].discard(c)
        done += 1
        if not pending[r]:                         # stream order: next sweep after the whole kernel
            sweep[r] += 1
            pending[r] = set(range(gx))
    return done, sweep


@pytest.mark.parametrize("world,gx", [(2, 1), (2, 5), (3, 4), (5, 3), (8, 6)])
def test_protocol_no_deadlock_and_exact_versions(world, gx):
    rng = random.Random(world * 100 + gx)
    sweeps = 6
    for _ in range(60):
        done, sweep = run_model(world, gx, sweeps, rng)
        assert done == world * gx * sweeps
        assert sweep == [sweeps + 1] * world


def test_protocol_needs_the_neighbouring_columns():
    """Waiting on column c alone is not enough: the halo a tile reads spans the
    neighbour's tiles c-1..c+1, so the narrow rule admits a schedule that reads
    stale (or already overwritten) halo data -- the model must catch it."""
    rng = random.Random(7)
    caught = 0
    for _ in range(200):
        try:
            run_model(2, 4, 4, rng, span=0)
        except AssertionError:
            caught += 1
    assert caught > 0


def test_neighbours():
    assert shard.neighbours(1, 0) == (None, None)
    assert shard.neighbours(3, 0) == (None, 1)
    assert shard.neighbours(3, 1) == (0, 2)
    assert shard.neighbours(3, 2) == (1, None)
