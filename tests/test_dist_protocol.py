"""CPU model of the device-side exchange of the distributed rounds, -m "not gpu".

k_persistent_dist keeps one color replica per part; every color word a part writes for one
of its own vertices also goes to the other replicas — with boundary filtering only to the
replicas of parts that own a neighbour of that vertex — and each part reads nothing but its
own replica. This model runs exactly that write/read discipline (one Jacobi round at a time,
per-part replicas, per-vertex masks) with the oracle's step functions for the per-vertex
arithmetic, and checks the colors assembled from the owners' replicas against the plain
oracle: filtered broadcasts lose no information any part ever reads.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from paper_conf_ipps_licqfsty16_b200 import gen
from tests._inputs import random_graph

LOW, PAP = oracle.TIEBREAK_LOWID_KEEPS, oracle.TIEBREAK_PAPER


def owner_of(ranges, w):
    return int(np.searchsorted(ranges, w, side="right") - 1)


def remote_masks(g, ranges, p):
    """bit q set iff part q (q != p) owns a neighbour of v, for v owned by p."""
    lo, hi = ranges[p], ranges[p + 1]
    masks = np.zeros(hi - lo, np.int64)
    for v in range(lo, hi):
        m = 0
        for w in g.col_idx[g.row_ptr[v]:g.row_ptr[v + 1]]:
            m |= 1 << owner_of(ranges, int(w))
        masks[v - lo] = m & ~(1 << p)
    return masks


def device_exchange_model(g, ranges, tb, use_masks):
    P = len(ranges) - 1
    n = g.n
    masks = [remote_masks(g, ranges, p) if use_masks else None for p in range(P)]
    rep = np.zeros((P, n), np.int32)  # every replica starts uncolored
    W = [np.arange(ranges[p], ranges[p + 1], dtype=np.int32) for p in range(P)]
    rounds = 0
    while sum(len(w) for w in W):
        rounds += 1
        # assignment against each part's own replica (Jacobi: the round's snapshot)
        writes = []
        for p in range(P):
            tent = oracle.assign(g, W[p], rep[p]) if len(W[p]) else np.zeros(0, np.int32)
            writes.append((p, W[p], tent))
        # stores: own replica always, other replicas only if they own a neighbour
        for p, wl, tent in writes:
            for v, c in zip(wl, tent):
                rep[p, v] = c
                m = masks[p][v - ranges[p]] if use_masks else ~(1 << p)
                for q in range(P):
                    if q != p and (int(m) >> q) & 1:
                        rep[q, v] = c
        # detection of each part's vertices against its own replica (after the barrier)
        W = [wl[oracle.detect(g, wl, rep[p], tb).astype(bool)] if len(wl) else wl
             for p, wl in enumerate(W)]
    colors = np.zeros(n, np.int32)
    for p in range(P):  # assembled range by range from the owners' replicas
        colors[ranges[p]:ranges[p + 1]] = rep[p, ranges[p]:ranges[p + 1]]
    return colors, rounds


@pytest.mark.parametrize("seed", range(10))
@pytest.mark.parametrize("P", [2, 3, 5])
def test_filtered_broadcast_equals_oracle(seed, P):
    g = random_graph(seed, n=120) if seed < 6 else gen.stencil3d(6, 5, 4 + seed, 27)
    rng = np.random.default_rng(seed)
    cuts = np.sort(rng.integers(0, g.n + 1, P - 1))
    ranges = np.concatenate([[0], cuts, [g.n]]).astype(np.int64)
    for tb in (LOW, PAP):
        ref = oracle.jacobi(g, tb)
        for use_masks in (False, True):
            colors, rounds = device_exchange_model(g, ranges, tb, use_masks)
            assert rounds == ref.rounds and np.array_equal(colors, ref.colors), (use_masks, tb)


def test_masks_skip_interior_vertices_of_slabs():
    """A z-slab partition of a 27-point stencil: only the planes next to a cut are boundary
    vertices (2P/N of the planes), so most stores stay local."""
    g = gen.stencil3d(6, 6, 12, 27)
    ranges = np.array([0, 6 * 6 * 6, g.n], np.int64)
    m0 = remote_masks(g, ranges, 0)
    assert (m0 != 0).sum() == 36  # the last plane of part 0
    assert set(np.unique(m0)) == {0, 2}
