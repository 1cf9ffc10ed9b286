"""Schedule oracle: the CTA-clustering partition written out from its definition.

TEST INFRASTRUCTURE ONLY.  Only tests/, ``__graft_entry__.smoke()`` and
bench.py's cpu_baseline / ``--impl reference`` legs may import this module.  It
shares no code with the CUDA path (``paper_conf_asplos_lis0l0c17_b200``) and
imports nothing from it.

What it follows (§4.2 "CTA Clustering"):

* Step 1, partitioning ``f: O -> C`` (Eq. 2-5): the CTAs of the
  original kernel are put in the order given by a CTA *indexing method*
  (Fig. 7: row-major = "Y-partitioning", column-major =
  "X-partitioning", tile-wise, or an arbitrary user order) and the ordered
  list is cut into ``M`` balanced contiguous chunks.  Eq. 3 covers
  ``M | |V|``; Eq. 4/5 extend it so the chunks are "as balanced as possible".
  The printed conditions of Eq. 4/5 are garbled (readings R1/R2);
  this oracle does NOT evaluate them.  It states the balance rule directly:
  the first ``|V| % M`` chunks hold ``|V|//M + 1`` CTAs, the rest ``|V|//M``
  (the reading that Eq. 7 and Listing 5's ``_jobs = _cd + (sm_id < _ck)``,
  P:2187 l.14, both imply), then finds ``(w, i)`` for a position by walking the
  chunk boundaries.
* Step 2, inverting ``f^-1: C -> O`` (Eq. 6/7): here the inverse
  is taken as the literal table inverse of step 1, not via Eq. 7, so that the
  closed form can be *checked* against it in tests.
* Tile-wise indexing (Fig. 7 tile panel, garbled at P:1891-1919): reading R6 --
  tiles of ``tile_w x tile_h`` CTAs visited in row-major tile order, CTAs
  row-major inside each tile, edge tiles clipped.

Identifiers: ``v`` is a CTA's *position* in the chosen order (the paper's
``v``); the library's tables are keyed by the CTA's row-major linear id
``lin = by * gx + bx`` so that censuses are order-independent.
"""
from __future__ import annotations

import numpy as np

ROW, COL, TILE, USER = 0, 1, 2, 3


def order_sequence(gx: int, gy: int, order: int, tile_w: int = 1, tile_h: int = 1,
                   user_order=None) -> np.ndarray:
    """Return ``seq`` with ``seq[v] = lin`` (row-major id) of the CTA at position v.

    Built by sorting every CTA by the indexing method's sort key (Fig. 7).
    """
    by, bx = np.divmod(np.arange(gx * gy, dtype=np.int64), gx)
    lin = by * gx + bx
    if order == ROW:            # v = blockIdx.y * gridDim.x + blockIdx.x
        keys = (bx, by)         # np.lexsort: last key is primary
    elif order == COL:          # v = blockIdx.x * gridDim.y + blockIdx.y
        keys = (by, bx)
    elif order == TILE:         # tiles row-major, CTAs row-major inside a tile (R6)
        if tile_w < 1 or tile_h < 1:
            raise ValueError("tile dims must be >= 1")
        keys = (bx, by, bx // tile_w, by // tile_h)
    elif order == USER:         # arbitrary order supplied as rank -> lin
        u = np.asarray(user_order, dtype=np.int64)
        if u.shape != (gx * gy,) or not np.array_equal(np.sort(u), lin):
            raise ValueError("user_order must be a permutation of range(gx*gy)")
        return u.copy()
    else:
        raise ValueError(f"unknown order {order}")
    return lin[np.lexsort(keys)]


def cluster_sizes(V: int, M: int) -> np.ndarray:
    """Balanced chunk sizes: the first V % M chunks get one extra CTA."""
    q, r = divmod(V, M)
    return np.array([q + 1] * r + [q] * (M - r), dtype=np.int64)


def plan(gx: int, gy: int, order: int, M: int, tile_w: int = 1, tile_h: int = 1,
         user_order=None) -> dict:
    """The whole partition: perm (cluster-major list of lin ids), offsets[M+1], q, r."""
    if gx < 0 or gy < 0 or M < 1:
        raise ValueError("bad grid / M")
    seq = order_sequence(gx, gy, order, tile_w, tile_h, user_order)
    V = gx * gy
    sizes = cluster_sizes(V, M)
    offsets = np.zeros(M + 1, dtype=np.int64)
    offsets[1:] = np.cumsum(sizes)
    # clusters are contiguous chunks of the ordered list, so the cluster-major
    # list of tasks is the ordered list itself, cut at ``offsets``.
    return {"V": V, "M": M, "q": V // M, "r": V % M,
            "perm": seq.astype(np.int32), "offsets": offsets.astype(np.int32)}


def f(V: int, M: int, v: int) -> tuple[int, int]:
    """Partition f(v) = (w, i): walk the chunk boundaries (no closed form)."""
    start = 0
    for i, size in enumerate(cluster_sizes(V, M)):
        if v < start + size:
            return int(v - start), i
        start += size
    raise ValueError("v out of range")


def f_inv(V: int, M: int, w: int, i: int) -> int:
    """Inverting f^-1(w, i) = v as the table inverse of ``f``."""
    sizes = cluster_sizes(V, M)
    if not (0 <= i < M and 0 <= w < sizes[i]):
        raise ValueError("(w, i) not in any cluster")
    return int(sizes[:i].sum() + w)


def rd_binding(u: int, M: int) -> tuple[int, int]:
    """Eq. 8 RR-based binding: (w, i) = (u / M, u % M)."""
    return u // M, u % M


def rd_redirect(V: int, M: int, u: int) -> int:
    """Redirection-based clustering, Listing 4 l.4, the paper's own
    definition of RD (binding + inverting in one line):
        v = (u % SM) * (_ctas / SM + 1) + u / SM + min(0, (_ctas % SM) - (u % SM))
    Kept literally: for clusters of size q the last Eq. 8 slot spills into the
    next cluster's first slot, which is what makes Listing 4 a bijection."""
    return (u % M) * (V // M + 1) + u // M + min(0, (V % M) - (u % M))


def expected_census(V: int) -> np.ndarray:
    """Every logical CTA runs exactly once (the orderless property)."""
    return np.ones(V, dtype=np.uint32)
