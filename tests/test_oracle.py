"""Pins for the CPU oracle (oracle/), -m "not gpu".

The oracle is pinned to things other than itself:
  * O1 (Algorithm 1) == networkx.greedy_color in natural order, +1 (library routine);
  * hand-derived traces (tests/golden/hand_traces.json) for both tie-break rules;
  * closed-form round counts / color counts on natural-order paths and grids;
  * brute-force chromatic numbers on tiny graphs (colors >= chi; min over orders == chi);
  * the id-reversal relation Jacobi_paper(G) = rev(Jacobi_lowid(rev(G))) [derived];
  * invariants: proper coloring, color <= deg+1, W strictly shrinking, R <= n;
  * two independent implementations (C liboracle vs pure-Python pyoracle) agree.
"""
from __future__ import annotations

import itertools
import json
import os

import networkx as nx
import numpy as np
import pytest

import oracle
from oracle import pyoracle
from paper_conf_ipps_licqfsty16_b200 import gen
from tests._inputs import adjacency, random_graph, raw_csr, reverse_ids, with_loops_and_dups

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "hand_traces.json")
LOW, PAP = oracle.TIEBREAK_LOWID_KEEPS, oracle.TIEBREAK_PAPER


def to_nx(g):
    G = nx.Graph()
    G.add_nodes_from(range(g.n))
    for v in range(g.n):
        for w in g.col_idx[g.row_ptr[v]:g.row_ptr[v + 1]]:
            G.add_edge(v, int(w))
    return G


def is_proper(g, colors):
    for v in range(g.n):
        for w in g.col_idx[g.row_ptr[v]:g.row_ptr[v + 1]]:
            if w != v and colors[v] == colors[w]:
                return False
    return True


# ----------------------------------------------------------------------------- O1
@pytest.mark.parametrize("seed", range(60))
def test_alg1_matches_networkx_natural_order(seed):
    g = random_graph(seed)
    ours = oracle.alg1(g)
    G = to_nx(g)
    ref = nx.greedy_color(G, strategy=lambda G_, c: range(g.n))
    assert [ref[v] + 1 for v in range(g.n)] == ours.tolist()


def test_alg1_matches_networkx_rmat_s12():
    g = gen.rmat(12, 8, 0.57, 0.19, 0.19, seed=11)
    ref = nx.greedy_color(to_nx(g), strategy=lambda G_, c: range(g.n))
    assert np.array_equal(oracle.alg1(g), np.array([ref[v] + 1 for v in range(g.n)]))


def test_alg1_bipartite_and_grids_natural_order():
    # natural-order greedy on a path / 5-pt / 7-pt grid is the checkerboard 2-coloring;
    # the 9-pt and 27-pt box stencils take 4 and 8 colors (2^d parity classes).
    assert oracle.alg1(gen.from_edges(7, [(i, i + 1) for i in range(6)])).max() == 2
    assert oracle.alg1(gen.stencil2d(9, 7, 5)).max() == 2
    assert oracle.alg1(gen.stencil3d(5, 6, 7, 7)).max() == 2
    assert oracle.alg1(gen.stencil2d(9, 7, 9)).max() == 4
    assert oracle.alg1(gen.stencil3d(5, 6, 7, 27)).max() == 8


# ----------------------------------------------------------------------------- golden
def load_cases():
    with open(GOLDEN) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", load_cases(), ids=lambda c: c["name"])
@pytest.mark.parametrize("rule", ["lowid", "paper"])
def test_hand_traces(case, rule):
    g = gen.from_edges(case["n"], case["edges"])
    tb = LOW if rule == "lowid" else PAP
    exp = case[rule]
    res = oracle.jacobi(g, tb)
    assert res.converged
    assert res.rounds == len(exp["worklists"])
    assert res.colors.tolist() == exp["history"][-1]
    assert res.round_sizes.tolist() == [len(w) for w in exp["worklists"]]
    # colors after every round, via the bounded-rounds entry point
    for r, hist in enumerate(exp["history"], start=1):
        part = oracle.jacobi(g, tb, max_rounds=r)
        assert part.colors.tolist() == hist, (r, part.colors.tolist(), hist)
    # the pure-Python twin reproduces the worklists themselves
    col, rounds, wls, history = pyoracle.jacobi(case["n"], adjacency(g),
                                                pyoracle.LOWID_KEEPS if rule == "lowid"
                                                else pyoracle.PAPER)
    assert wls == exp["worklists"] and history == exp["history"]
    assert oracle.alg1(g).tolist() == case["alg1"]


@pytest.mark.parametrize("n", [1, 2, 3, 5, 9, 17])
def test_complete_graph(n):
    g = gen.from_edges(n, [(i, j) for i in range(n) for j in range(i + 1, n)])
    lo = oracle.jacobi(g, LOW)
    pa = oracle.jacobi(g, PAP)
    assert lo.rounds == n and pa.rounds == n
    assert lo.colors.tolist() == list(range(1, n + 1))
    assert pa.colors.tolist() == list(range(n, 0, -1))
    assert lo.round_sizes.tolist() == list(range(n, 0, -1))


# ----------------------------------------------------------------------------- closed forms
@pytest.mark.parametrize("n", [1, 2, 3, 4, 7, 16, 31])
def test_path_rounds_closed_form(n):
    g = gen.from_edges(n, [(i, i + 1) for i in range(n - 1)])
    for tb in (LOW, PAP):
        res = oracle.jacobi(g, tb)
        assert res.rounds == n
        assert res.num_colors == (1 if n == 1 else 2)
    assert np.array_equal(oracle.jacobi(g, LOW).colors, oracle.alg1(g))


@pytest.mark.parametrize("N", [2, 3, 5, 8, 11])
def test_grid_round_closed_forms(N):
    # natural-order grids (SURVEY §4 closed forms, from an independent simulator):
    # 5-pt N x N -> 2N-1 rounds; 7-pt N^3 -> 3N-2; 27-pt N^3 -> 3N+2 (N even) / 3N (N odd);
    # 9-pt N x N -> 2N-1 (N odd) / 2N (N even). Both rules; colors 2, 2, 8, 4;
    # lowid == Algorithm 1 on all of them.
    cases = [(gen.stencil2d(N, N, 5), 2 * N - 1, 2),
             (gen.stencil3d(N, N, N, 7), 3 * N - 2, 2),
             (gen.stencil3d(N, N, N, 27), 3 * N + 2 if N % 2 == 0 else 3 * N, 8),
             (gen.stencil2d(N, N, 9), 2 * N if N % 2 == 0 else 2 * N - 1, 4)]
    for g, rounds, colors in cases:
        a1 = oracle.alg1(g)
        for tb in (LOW, PAP):
            res = oracle.jacobi(g, tb)
            assert res.rounds == rounds, (g.name, tb, res.rounds)
            assert res.num_colors == colors, (g.name, tb)
        assert np.array_equal(oracle.jacobi(g, LOW).colors, a1), g.name


def test_nnz_zero_and_empty():
    g = gen.from_edges(5, np.zeros((0, 2), np.int64))
    res = oracle.jacobi(g, LOW)
    assert res.rounds == 1 and res.colors.tolist() == [1] * 5
    g0 = gen.from_edges(0, np.zeros((0, 2), np.int64))
    res0 = oracle.jacobi(g0, LOW)
    assert res0.rounds == 0 and len(res0.colors) == 0
    assert len(oracle.alg1(g0)) == 0


# ----------------------------------------------------------------------------- brute force
def chromatic_number(n, adj):
    for k in range(1, n + 1):
        for assignment in itertools.product(range(k), repeat=n):
            if all(assignment[v] != assignment[w] for v in range(n) for w in adj[v] if w != v):
                return k
    return 0


@pytest.mark.parametrize("seed", range(25))
def test_brute_force_chromatic_bounds(seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(1, 8))
    g = random_graph(1000 + seed, n=n)
    adj = adjacency(g)
    chi = chromatic_number(n, adj)
    best = min(max(pyoracle.greedy(n, adj, order)) for order in itertools.permutations(range(n)))
    assert best == chi  # some order makes greedy optimal
    assert oracle.alg1(g).max() >= chi
    for tb in (LOW, PAP):
        assert oracle.jacobi(g, tb).num_colors >= chi


# ----------------------------------------------------------------------------- relations
@pytest.mark.parametrize("seed", range(40))
def test_reversal_relation_and_invariants(seed):
    g = random_graph(seed)
    lo = oracle.jacobi(g, LOW)
    pa = oracle.jacobi(g, PAP)
    lo_rev = oracle.jacobi(reverse_ids(g), LOW)
    assert np.array_equal(pa.colors, lo_rev.colors[::-1])
    assert pa.rounds == lo_rev.rounds
    deg = g.degrees
    for res in (lo, pa):
        assert res.converged
        assert is_proper(g, res.colors)
        assert np.all(res.colors >= 1) and np.all(res.colors <= deg + 1)
        assert res.rounds <= max(g.n, 0)
        ws = res.trace["w_size"]
        nx_ = res.trace["next_size"]
        assert np.all(nx_ < ws)                 # W_{r+1} strictly inside W_r
        assert np.array_equal(ws[1:], nx_[:-1])  # the trace chains
        if len(nx_):
            assert nx_[-1] == 0
        assert int(res.trace["max_color"][-1]) == res.num_colors


@pytest.mark.parametrize("seed", range(40))
def test_c_oracle_equals_python_twin(seed):
    g = random_graph(seed)
    adj = adjacency(g)
    for tb, rule in ((LOW, pyoracle.LOWID_KEEPS), (PAP, pyoracle.PAPER)):
        res = oracle.jacobi(g, tb)
        col, rounds, wls, _ = pyoracle.jacobi(g.n, adj, rule)
        assert res.colors.tolist() == col and res.rounds == rounds
        assert res.round_sizes.tolist() == [len(w) for w in wls]
    assert oracle.alg1(g).tolist() == pyoracle.greedy(g.n, adj)


@pytest.mark.parametrize("seed", range(20))
def test_detect_over_v_equals_over_w(seed):
    g = random_graph(seed)
    for tb in (LOW, PAP):
        a = oracle.jacobi(g, tb, detect_over_v=True)
        b = oracle.jacobi(g, tb, detect_over_v=False)
        assert np.array_equal(a.colors, b.colors) and a.rounds == b.rounds
        assert np.array_equal(a.trace, b.trace)


@pytest.mark.parametrize("seed", range(20))
def test_self_loops_and_duplicates_do_not_matter(seed):
    g = random_graph(seed)
    h = with_loops_and_dups(g, seed)
    for tb in (LOW, PAP):
        a = oracle.jacobi(g, tb)
        b = oracle.jacobi(h, tb)
        assert np.array_equal(a.colors, b.colors) and a.rounds == b.rounds
        assert np.array_equal(a.round_sizes, b.round_sizes)
    assert np.array_equal(oracle.alg1(g), oracle.alg1(h))


@pytest.mark.parametrize("seed", range(12))
def test_partitioned_equals_plain(seed):
    g = random_graph(seed)
    rng = np.random.default_rng(seed)
    for tb in (LOW, PAP):
        ref = oracle.jacobi(g, tb)
        for P in (1, 2, 3, 5):
            cuts = np.sort(rng.integers(0, g.n + 1, P - 1))
            ranges = np.concatenate([[0], cuts, [g.n]]).astype(np.int64)
            col, rounds = oracle.jacobi_partitioned(g, P, tb, ranges)
            assert np.array_equal(col, ref.colors) and rounds == ref.rounds
            col2, _ = oracle.jacobi_partitioned(g, P, tb)
            assert np.array_equal(col2, ref.colors)


def test_threads_do_not_change_result():
    g = gen.rmat(13, 8, 0.57, 0.19, 0.19, seed=5)
    for tb in (LOW, PAP):
        a = oracle.jacobi(g, tb, nthreads=1)
        b = oracle.jacobi(g, tb, nthreads=4)
        assert np.array_equal(a.colors, b.colors) and np.array_equal(a.trace, b.trace)


@pytest.mark.parametrize("seed", range(15))
def test_step_functions(seed):
    g = random_graph(seed)
    adj = adjacency(g)
    rng = np.random.default_rng(seed)
    snap = rng.integers(0, 6, g.n).astype(np.int32)
    wl = np.sort(rng.choice(g.n, size=int(rng.integers(0, g.n + 1)), replace=False)).astype(np.int32)
    tent = oracle.assign(g, wl, snap)
    for i, v in enumerate(wl):
        assert tent[i] == pyoracle.mex_positive({int(snap[w]) for w in adj[int(v)]})
    for tb, rule in ((LOW, pyoracle.LOWID_KEEPS), (PAP, pyoracle.PAPER)):
        fl = oracle.detect(g, wl, snap, tb)
        for i, v in enumerate(wl):
            v = int(v)
            exp = any(snap[w] == snap[v] and pyoracle.loses(rule, v, w) for w in adj[v])
            assert bool(fl[i]) == exp


def test_step_assign_self_loop_reading_c7():
    """Reading C7 on the step API: oracle_assign is Alg. 5 l.5-6 literally —
    w ranges over every listed entry, so a self-loop forbids v's own snapshot color. Hand
    values: a lone vertex with a loop and snapshot color 1 gets 2 (without the loop: 1); a
    duplicated entry changes nothing; detection never flags a loop (l.14: v < v is false)."""
    loop = raw_csr(1, [(0, 0)])
    assert oracle.assign(loop, [0], [1]).tolist() == [2]
    assert oracle.assign(loop, [0], [3]).tolist() == [1]
    bare = raw_csr(1, [])
    assert oracle.assign(bare, [0], [1]).tolist() == [1]
    # path 0-1 with a loop on 1 and a duplicated (0,1): snapshot [1, 2]
    g = raw_csr(2, [(0, 1), (0, 1), (1, 0), (1, 0), (1, 1)])
    assert oracle.assign(g, [0, 1], [1, 2]).tolist() == [1, 3]
    assert oracle.detect(g, [0, 1], [2, 2], LOW).tolist() == [0, 1]
    assert oracle.detect(loop, [0], [1], LOW).tolist() == [0]
    assert oracle.detect(loop, [0], [1], PAP).tolist() == [0]


def test_rmat_s16_quality_and_rule_asymmetry():
    """cfg1: lowid uses about as many colors as Algorithm 1 (north_star: within 10%),
    the paper rule noticeably more on unpermuted R-MAT (SURVEY exec. summary item 3)."""
    g = gen.config(1)
    a1 = int(oracle.alg1(g).max())
    lo = oracle.jacobi(g, LOW)
    pa = oracle.jacobi(g, PAP)
    assert abs(lo.num_colors - a1) <= 0.10 * a1
    assert pa.num_colors > lo.num_colors
    assert is_proper(g, lo.colors) and is_proper(g, pa.colors)


# ----------------------------------------------------------------------------- O3 (§8(f) item 4)
def path(n):
    return gen.from_edges(n, np.stack([np.arange(n - 1), np.arange(1, n)], 1).astype(np.int64))


@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("part", [0, 1])
def test_gs_one_substep_is_jacobi(seed, part):
    """K = 1: one sub-step per round is O2 exactly (colors, R, the whole trace)."""
    g = random_graph(seed) if seed < 10 else gen.rmat(11, 8, 0.57, 0.19, 0.19, seed=seed)
    for tb in (LOW, PAP):
        a = oracle.gauss_seidel(g, 1, part, tb)
        b = oracle.jacobi(g, tb)
        assert np.array_equal(a.colors, b.colors) and a.rounds == b.rounds
        assert np.array_equal(a.trace, b.trace)


@pytest.mark.parametrize("seed", range(10))
def test_gs_n_substeps_is_algorithm1(seed):
    """K = n: every vertex is its own sub-step, taken in id order (blocked, and strided since
    v mod n = v), i.e. Algorithm 1 in natural order — pinned to networkx's greedy_color —
    finished in one round (a sequential greedy coloring has no conflict)."""
    g = random_graph(seed, n=40)
    G = to_nx(g)
    nxc = nx.greedy_color(G, strategy=lambda G_, c: list(range(g.n)))
    ref = np.array([nxc[v] + 1 for v in range(g.n)], np.int32)
    for part in (0, 1):
        for tb in (LOW, PAP):
            r = oracle.gauss_seidel(g, max(g.n, 1), part, tb)
            assert np.array_equal(r.colors, ref) and r.rounds == (1 if g.n else 0)


def test_gs_hand_traces():
    """Hand-derived. P4 = 0-1-2-3:
    K=2 strided, lowid: sub-step {0,2} against all-0 -> [1,0,1,0]; {1,3} -> [1,2,1,2]; proper, R=1.
    K=2 blocked ({0,1},{2,3}), lowid: {0,1} -> [1,1,0,0]; {2,3} against it: 2 -> mex{1,0}=2,
      3 -> mex{0}=1 -> [1,1,2,1]; 1 loses to 0 -> W2={1}; round 2: 1 -> mex{1,2}=3 -> [1,3,2,1], R=2.
    K=2 blocked, paper rule: same round 1; 0 loses to 1 (0 < 1) -> W2={0}; 0 -> mex{1}=2 -> [2,1,2,1].
    K3, K=3 strided: 0 -> 1; 1 -> mex{1,0}=2; 2 -> mex{1,2}=3 -> [1,2,3], R=1."""
    p4 = path(4)
    r = oracle.gauss_seidel(p4, 2, 0, LOW)
    assert r.colors.tolist() == [1, 2, 1, 2] and r.rounds == 1
    r = oracle.gauss_seidel(p4, 2, 1, LOW)
    assert r.colors.tolist() == [1, 3, 2, 1] and r.rounds == 2
    assert r.round_sizes.tolist() == [4, 1]
    r = oracle.gauss_seidel(p4, 2, 1, PAP)
    assert r.colors.tolist() == [2, 1, 2, 1] and r.rounds == 2
    k3 = gen.from_edges(3, np.array([[0, 1], [1, 2], [0, 2]], np.int64))
    r = oracle.gauss_seidel(k3, 3, 0, LOW)
    assert r.colors.tolist() == [1, 2, 3] and r.rounds == 1


@pytest.mark.parametrize("n", [2, 5, 64, 1001])
def test_gs_path_two_strided_substeps_closed_form(n):
    """A natural-order path with K = 2 strided: evens take 1, then odds take 2 -> Algorithm 1
    (alternating 1, 2) in one round, against O2's n rounds (test_path_rounds_closed_form)."""
    r = oracle.gauss_seidel(path(n), 2, 0, LOW)
    assert r.rounds == 1 and r.colors.tolist() == [1 + (v & 1) for v in range(n)]


@pytest.mark.parametrize("seed", range(24))
def test_gs_c_equals_python_twin_and_invariants(seed):
    g = random_graph(seed)
    adj = adjacency(g)
    rng = np.random.default_rng(seed)
    K = int(rng.integers(2, 7))
    for part in (0, 1):
        for tb, rule in ((LOW, pyoracle.LOWID_KEEPS), (PAP, pyoracle.PAPER)):
            r = oracle.gauss_seidel(g, K, part, tb)
            col, R, wls = pyoracle.gauss_seidel(g.n, adj, K, part, rule)
            assert r.colors.tolist() == col and r.rounds == R
            assert r.round_sizes.tolist() == [len(w) for w in wls]
            assert is_proper(g, r.colors)
            assert np.all(r.colors <= g.degrees + 1) and (g.n == 0 or r.colors.min() >= 1)
            for a, b in zip(wls, wls[1:]):  # W strictly shrinking, W_{r+1} inside W_r
                assert len(b) < len(a) and set(b) <= set(a)
