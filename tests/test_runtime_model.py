"""CPU model of the agent scheduler protocol (csrc/cc_runtime.cuh: lane0_next,
steal_scan, producer_next) under random interleavings of the agents' atomic
operations (SURVEY.md §4 "Agent-runtime model").  Every slot of every cluster
queue must be claimed exactly once and every agent must terminate, for any
number of agents per cluster (including clusters with none), any batch size,
with the speculative next-batch claim and the early-exit `claimed` count.

This is a model of the host-visible protocol, not of the arithmetic; the GPU
census tests check the real kernels."""
import random

import pytest


class Shared:
    def __init__(self, sizes):
        self.head = [0] * len(sizes)
        self.size = list(sizes)
        self.claimed = 0
        self.V = sum(sizes)


def agent(sh: Shared, home: int, batch: int, steal: bool, out: list):
    """Generator: yields between atomic operations (the interleaving points)."""
    M = len(sh.size)
    q, bq, bw, be, spec, mine = home, -1, 0, 0, None, 0
    while True:
        if bw < be:
            out.append((bq, bw))
            bw += 1
            continue
        # lane0_next
        got = None
        while got is None:
            if spec is not None:
                sq, w = spec
                spec = None
            elif q >= 0:
                sq = q
                w = sh.head[sq]; sh.head[sq] += batch          # atomic fetch-add
                yield
            else:
                return
            if w < sh.size[sq]:
                bq, bw, be = sq, w, min(w + batch, sh.size[sq])
                mine += be - w
                if w + batch < sh.size[sq]:                     # speculative next claim
                    spec = (sq, sh.head[sq]); sh.head[sq] += batch
                    yield
                got = True
            elif sq == q:
                if not steal:
                    return
                old = sh.claimed; sh.claimed += mine            # value-returning add
                allc = old + mine
                mine = 0
                yield
                if allc >= sh.V:
                    return
                # warp-parallel scan, nearest first from home
                cand = [(home + 1 + k) % M for k in range(M)]
                avail = [c for c in cand if sh.head[c] < sh.size[c]]
                yield
                if not avail:
                    return
                q = avail[0]
                spec = None


def run(sizes, agents_per_queue, batch, steal, seed):
    rng = random.Random(seed)
    sh = Shared(sizes)
    out = []
    gens = [agent(sh, h, batch, steal, out) for h, n in enumerate(agents_per_queue) for _ in range(n)]
    live = list(gens)
    steps = 0
    while live:
        g = rng.choice(live)
        try:
            next(g)
        except StopIteration:
            live.remove(g)
        steps += 1
        assert steps < 10 ** 6
    return out


@pytest.mark.parametrize("seed", range(40))
def test_exactly_once_with_stealing(seed):
    rng = random.Random(1000 + seed)
    M = rng.randint(1, 12)
    sizes = [rng.randint(0, 30) for _ in range(M)]
    agents = [rng.randint(0, 3) for _ in range(M)]
    if sum(agents) == 0:
        agents[rng.randrange(M)] = 1
    batch = rng.randint(1, 5)
    out = run(sizes, agents, batch, True, seed)
    expect = sorted((q, w) for q, s in enumerate(sizes) for w in range(s))
    assert sorted(out) == expect                      # every slot exactly once


@pytest.mark.parametrize("seed", range(10))
def test_without_stealing_only_home_clusters_run(seed):
    """steal = 0 (the paper's static binding): clusters with agents run exactly
    once; clusters without any agent are not run at all (P:2207's hazard)."""
    rng = random.Random(seed)
    M = 6
    sizes = [rng.randint(1, 20) for _ in range(M)]
    agents = [rng.randint(0, 2) for _ in range(M)]
    out = run(sizes, agents, rng.randint(1, 4), False, seed)
    expect = sorted((q, w) for q, s in enumerate(sizes) if agents[q] for w in range(s))
    assert sorted(out) == expect
