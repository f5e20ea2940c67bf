"""Seeded small-graph families for tests (input generation only — no coloring arithmetic).

Everything goes through the shared generator module (paper_conf_ipps_licqfsty16_b200.gen),
except `raw_csr`, which deliberately keeps self-loops and duplicate entries to exercise
readings C7/C9.
"""
from __future__ import annotations

import numpy as np

from paper_conf_ipps_licqfsty16_b200 import gen


def random_graph(seed: int, n: int | None = None, kind: str | None = None):
    rng = np.random.default_rng(seed)
    if n is None:
        n = int(rng.integers(1, 60))
    kinds = ["er", "hub", "dense", "sparse", "clique+path", "bipartite"]
    kind = kind or kinds[seed % len(kinds)]
    if kind == "er":
        m = int(rng.integers(0, 3 * n + 1))
        e = rng.integers(0, n, size=(m, 2))
    elif kind == "hub":  # a few hubs + random edges, isolated vertices likely
        hubs = rng.integers(0, n, size=max(1, n // 10))
        m = int(rng.integers(n, 4 * n + 1))
        e = np.stack([rng.choice(hubs, m), rng.integers(0, n, m)], 1)
    elif kind == "dense":
        p = rng.uniform(0.3, 0.9)
        iu = np.triu_indices(n, 1)
        keep = rng.random(len(iu[0])) < p
        e = np.stack([iu[0][keep], iu[1][keep]], 1)
    elif kind == "sparse":
        m = int(rng.integers(0, n + 1))
        e = rng.integers(0, n, size=(m, 2))
    elif kind == "clique+path":
        k = min(n, int(rng.integers(1, 12)))
        iu = np.triu_indices(k, 1)
        cl = np.stack(iu, 1)
        path = np.stack([np.arange(k, n - 1), np.arange(k + 1, n)], 1) if n - 1 > k else \
            np.zeros((0, 2), np.int64)
        e = np.concatenate([cl, path]) if len(path) else cl
        perm = rng.permutation(n)
        e = perm[e] if len(e) else e
    elif kind == "bipartite":
        side = rng.random(n) < 0.5
        m = int(rng.integers(0, 3 * n + 1))
        a = rng.integers(0, n, m)
        b = rng.integers(0, n, m)
        keep = side[a] != side[b]
        e = np.stack([a[keep], b[keep]], 1)
    else:
        raise ValueError(kind)
    return gen.from_edges(n, np.asarray(e, np.int64).reshape(-1, 2))


def raw_csr(n: int, entries):
    """Directed CSR straight from (v, w) entries, rows sorted, loops and dups KEPT."""
    entries = sorted((int(v), int(w)) for v, w in entries)
    rp = np.zeros(n + 1, np.int64)
    for v, _ in entries:
        rp[v + 1] += 1
    rp = np.cumsum(rp).astype(np.int64)
    ci = np.array([w for _, w in entries], np.int32)
    return gen.Graph(n, len(ci), rp, ci, "raw")


def with_loops_and_dups(g, seed: int):
    """Same pattern as g plus self-loops on some vertices and duplicated entries (kept sym)."""
    rng = np.random.default_rng(seed)
    ent = []
    for v in range(g.n):
        for w in g.col_idx[g.row_ptr[v]:g.row_ptr[v + 1]]:
            ent.append((v, int(w)))
    extra = []
    for v, w in ent:
        if v < w and rng.random() < 0.3:
            extra += [(v, w), (w, v)]
    loops = [(v, v) for v in range(g.n) if rng.random() < 0.3]
    return raw_csr(g.n, ent + extra + loops + loops)


def adjacency(g):
    """dict-of-sets adjacency (for the pure-Python twin)."""
    adj = {v: set() for v in range(g.n)}
    for v in range(g.n):
        for w in g.col_idx[g.row_ptr[v]:g.row_ptr[v + 1]]:
            adj[v].add(int(w))
    return adj


def reverse_ids(g):
    """rev: v -> n-1-v, rebuilt as a sorted CSR."""
    n = g.n
    e = []
    for v in range(n):
        for w in g.col_idx[g.row_ptr[v]:g.row_ptr[v + 1]]:
            e.append((n - 1 - v, n - 1 - int(w)))
    return gen.from_edges(n, np.asarray(e, np.int64).reshape(-1, 2))
