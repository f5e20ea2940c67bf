"""Pure-Python twin of the oracle for tiny graphs — TEST INFRASTRUCTURE ONLY.

Written separately from sgr_oracle.c (sets instead of labelled colorMask arrays, dict
adjacency instead of CSR) so that a slip in one is unlikely to be repeated in the other.
Follows PAPER.md Algorithm 1 and Algorithm 5 with Jacobi rounds
(SURVEY §8(c) C1-C4).
"""
from __future__ import annotations

LOWID_KEEPS = 0
PAPER = 1


def adjacency(n, edges):
    adj = {v: set() for v in range(n)}
    for u, v in edges:
        adj[u].add(v)
        adj[v].add(u)
    return adj


def mex_positive(forbidden):
    """min{ i > 0 : i not in forbidden } (Alg. 1 l.6)."""
    c = 1
    while c in forbidden:
        c += 1
    return c


def greedy(n, adj, order=None):
    """Algorithm 1 in the given order (natural order by default)."""
    color = [0] * n
    for v in (range(n) if order is None else order):
        color[v] = mex_positive({color[w] for w in adj[v]})
    return color


def loses(rule, v, w):
    return v < w if rule == PAPER else v > w


def jacobi(n, adj, rule=LOWID_KEEPS):
    """Returns (colors, rounds, [sorted W_r for r = 1..R], [colors after round r])."""
    color = [0] * n
    W = list(range(n))
    worklists, history = [], []
    while W:
        worklists.append(sorted(W))
        snapshot = list(color)
        for v in W:
            color[v] = mex_positive({snapshot[w] for w in adj[v]})
        W = [v for v in W if any(color[w] == color[v] and loses(rule, v, w) for w in adj[v])]
        history.append(list(color))
    return color, len(worklists), worklists, history


def gauss_seidel(n, adj, K, partition=0, rule=LOWID_KEEPS):
    """K-sub-step rounds: the round's vertices go in K groups, in
    order; a group sees the colors the earlier groups of the round gave. Returns
    (colors, rounds, [sorted W_r])."""
    def part(v):
        return (v * K) // n if partition == 1 else v % K
    color = [0] * n
    W = list(range(n))
    worklists = []
    while W:
        worklists.append(sorted(W))
        for j in range(K):
            seen = dict(enumerate(color))
            for v in W:
                if part(v) == j:
                    color[v] = mex_positive({seen[w] for w in adj[v]})
        W = [v for v in W if any(color[w] == color[v] and loses(rule, v, w) for w in adj[v])]
    return color, len(worklists), worklists
