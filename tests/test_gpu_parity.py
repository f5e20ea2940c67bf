"""Parity of the CUDA path (libsgr.so through its C ABI) against the CPU oracle (-m gpu).

Bar: everything here is integer work, so colors, the round count R and the
per-round worklist sizes |W_r| must be BIT-EXACT; the worklists' order is unspecified, so
step-level compaction is compared as ordered output (sgr_compact is order-preserving) and
the fused path's worklists through their sizes and the final colors.
"""
from __future__ import annotations

import os

import numpy as np
import pytest

import oracle
from paper_conf_ipps_licqfsty16_b200 import gen
from tests._inputs import random_graph, raw_csr, with_loops_and_dups

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # the marker keeps these off the CPU suite
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402

LOW, PAP = oracle.TIEBREAK_LOWID_KEEPS, oracle.TIEBREAK_PAPER
RULE = {LOW: "lowid", PAP: "paper"}


def dev(g):
    return (torch.from_numpy(np.ascontiguousarray(g.row_ptr)).cuda(),
            torch.from_numpy(np.ascontiguousarray(g.col_idx)).cuda())


def check_full(g, tb, **kw):
    rp, ci = dev(g)
    res = sgr.color(rp, ci, RULE[tb], trace=True, **kw)
    ref = oracle.jacobi(g, tb, nthreads=oracle.max_threads())
    got = res.colors.cpu().numpy()
    assert res.stats["rounds"] == ref.rounds, (g.name, res.stats["rounds"], ref.rounds)
    if not np.array_equal(got, ref.colors):
        bad = np.nonzero(got != ref.colors)[0]
        raise AssertionError(f"{g.name}: {len(bad)} colors differ, first {bad[:8]} "
                             f"got {got[bad[:8]]} want {ref.colors[bad[:8]]}")
    assert np.array_equal(res.round_sizes, ref.round_sizes), g.name
    assert np.array_equal(res.round_edges, ref.trace["w_edges"]), g.name
    assert res.stats["num_colors"] == ref.num_colors
    assert res.stats["edges_scanned"] == ref.edges_scanned
    assert res.stats["vertices_processed"] == ref.vertices_processed
    return res, ref


# ----------------------------------------------------------------------------- full path
@pytest.mark.parametrize("seed", range(48))
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_random_small_graphs(seed, tb):
    check_full(random_graph(seed), tb)


@pytest.mark.parametrize("tb", [LOW, PAP])
def test_cfg1_rmat_s16_bit_exact(tb):
    res, ref = check_full(gen.config(1), tb)
    if tb == LOW:  # north_star quality target: within 10% of Algorithm 1
        a1 = int(oracle.alg1(gen.config(1)).max())
        assert abs(res.stats["num_colors"] - a1) <= 0.1 * a1


@pytest.mark.parametrize("maker", [
    lambda: gen.stencil3d(24, 24, 24, 27),
    lambda: gen.stencil3d(13, 11, 9, 7),
    lambda: gen.stencil2d(57, 31, 5),
    lambda: gen.stencil2d(40, 40, 9),
    lambda: gen.er(1 << 15, 8 << 15, seed=3),
    lambda: gen.rmat(15, 8, 0.57, 0.19, 0.19, seed=4, permute=True),
    lambda: gen.rmat(14, 10, 0.45, 0.15, 0.15, seed=2),   # rmat-g shape (Table I)
    lambda: gen.rmat(14, 10, 0.25, 0.25, 0.25, seed=2),   # rmat-er shape (Table I)
], ids=["s27-24", "s7", "s5", "s9", "er15", "rmat15-perm", "rmat-g14", "rmat-er14"])
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_generator_families(maker, tb):
    check_full(maker(), tb)


def degree_boundary_graph():
    """Stars whose centres have degrees at every bin boundary, plus cliques K_70 / K_300
    (first fits above 64 and 256; K_300 rows straddle 1024-aligned chunk boundaries)."""
    edges = []
    n = 0
    for d in [0, 1, 2, 31, 32, 33, 61, 62, 63, 64, 65, 255, 256, 257, 507, 508, 509, 1015, 1016,
              1017, 1019, 1020, 1021, 2040,
              2041, 2047, 2048, 2049, 4095, 4096, 4097, 9000]:
        c = n
        edges += [(c, c + 1 + i) for i in range(d)]
        n += d + 1
    for k in (70, 300):
        base = n
        edges += [(base + i, base + j) for i in range(k) for j in range(i + 1, k)]
        n += k
    # tie the pieces together so the stars' leaves also collide
    edges += [(i, i + 7) for i in range(0, n - 7, 5)]
    return gen.from_edges(n, np.asarray(edges, np.int64))


@pytest.mark.parametrize("tb", [LOW, PAP])
@pytest.mark.parametrize("bins", [(0, 0), (62, 62), (1, 1), (8, 64), (32, 256), (62, 256), (1, 2)])
@pytest.mark.parametrize("mode", ["persistent", "host"])
@pytest.mark.parametrize("bits", [16, 32])
def test_degree_bins_and_windows(tb, bins, mode, bits):
    check_full(degree_boundary_graph(), tb, bin_small_max=bins[0], bin_med_max=bins[1],
               loop_mode=mode, color_bits=bits)


@pytest.mark.parametrize("cap,bits", [(40, 32), (299, 32), (300, 16), (0, 16)])
def test_color_overflow_rerun(cap, bits):
    """A first fit above the 16-bit word's color range (lowered by the color_cap test hook)
    discards the packed run and redoes the coloring with plain int32 words: same result."""
    g = degree_boundary_graph()  # contains K_300: colors up to 300
    for tb in (LOW, PAP):
        res, _ = check_full(g, tb, color_cap=cap)
        assert res.stats["color_bits"] == bits, (cap, res.stats["color_bits"])


@pytest.mark.parametrize("k", [64, 257, 520, 1100])
def test_complete_graphs_large_mex(k):
    g = gen.from_edges(k, [(i, j) for i in range(k) for j in range(i + 1, k)])
    for bins in [(0, 0), (1, 1), (62, 256), (1, 2)]:
        res, _ = check_full(g, LOW, bin_small_max=bins[0], bin_med_max=bins[1])
        assert res.colors.cpu().numpy().tolist() == list(range(1, k + 1))


@pytest.mark.parametrize("k", [30, 31, 32])
@pytest.mark.parametrize("apex_low", [False, True])
@pytest.mark.parametrize("mapping", [0, 1, 2])
def test_bin0_colors_beyond_31(k, apex_low, mapping):
    """A K_k clique plus an apex adjacent to all of it: a row of <= 32 entries whose
    neighbours end up colored 1..k, so the apex's first fit is k + 1 — past the 31 colors
    the byte-gather bit masks of bin 0 hold (the exact rescan must take over), in both
    bin-0 mappings of the flat build and both rules."""
    n = k + 1
    apex = 0 if apex_low else k
    others = [v for v in range(n) if v != apex]
    edges = [(others[i], others[j]) for i in range(k) for j in range(i + 1, k)]
    edges += [(apex, v) for v in others]
    g = gen.from_edges(n, np.asarray(edges, np.int64))
    for tb in (LOW, PAP):
        res, _ = check_full(g, tb, flat_bin0=mapping)
        assert res.stats["num_colors"] == n


@pytest.mark.parametrize("seed", range(8))
def test_self_loops_and_duplicates(seed):
    g = random_graph(seed, n=200)
    h = with_loops_and_dups(g, seed)
    for tb in (LOW, PAP):
        a = sgr.color(*dev(g), RULE[tb]).colors.cpu().numpy()
        b = sgr.color(*dev(h), RULE[tb]).colors.cpu().numpy()
        assert np.array_equal(a, b)
        assert np.array_equal(b, oracle.jacobi(h, tb).colors)


def test_edge_cases_n0_n1_nnz0():
    g0 = gen.from_edges(0, np.zeros((0, 2), np.int64))
    r0 = sgr.color(*dev(g0))
    assert r0.stats["rounds"] == 0 and r0.colors.numel() == 0
    g1 = gen.from_edges(1, np.zeros((0, 2), np.int64))
    r1 = sgr.color(*dev(g1))
    assert r1.stats["rounds"] == 1 and r1.colors.cpu().tolist() == [1]
    g5 = gen.from_edges(5, np.zeros((0, 2), np.int64))
    r5 = sgr.color(*dev(g5), trace=True)
    assert r5.stats["rounds"] == 1 and r5.colors.cpu().tolist() == [1] * 5
    assert r5.round_sizes.tolist() == [5]
    loops = raw_csr(3, [(0, 0), (1, 1), (2, 2)])
    assert sgr.color(*dev(loops)).colors.cpu().tolist() == [1, 1, 1]


@pytest.mark.parametrize("mode", ["host", "graph", "persistent"])
@pytest.mark.parametrize("batch", [1, 3, 8, 32])
def test_loop_modes_and_batches(mode, batch):
    g = gen.config(1)
    rp, ci = dev(g)
    ref = sgr.color(rp, ci).colors
    res = sgr.color(rp, ci, loop_mode=mode, rounds_per_batch=batch)
    assert torch.equal(res.colors, ref)


def test_profile_mode_and_stats():
    g = gen.config(1)
    rp, ci = dev(g)
    res = sgr.color(rp, ci, profile=True)
    st = res.stats
    assert st["kernel_launches"]["first"] == 1
    assert st["kernel_launches"]["round"] == 1  # persistent: every round in one launch
    assert st["kernel_ms"]["round"] > 0
    assert sum(st["bin_edges"].values()) + g.nnz == st["edges_scanned"]
    assert all(v >= 0 for v in st["kernel_ms"].values())
    assert st["bytes_algorithmic"] == sum(st["kernel_bytes"].values())
    ref = oracle.jacobi(g, LOW)
    assert torch.equal(res.colors.cpu(), torch.from_numpy(ref.colors))


def test_deterministic_repeats():
    g = gen.rmat(16, 8, 0.57, 0.19, 0.19, seed=9, permute=True)
    rp, ci = dev(g)
    a = sgr.color(rp, ci).colors.clone()
    for _ in range(3):
        assert torch.equal(sgr.color(rp, ci).colors, a)


def test_max_rounds_enoconv():
    g = gen.from_edges(6, [(i, i + 1) for i in range(5)])  # path: R = 6
    rp, ci = dev(g)
    with pytest.raises(RuntimeError, match="max_rounds"):
        sgr.color(rp, ci, max_rounds=3)
    assert sgr.color(rp, ci, max_rounds=6).stats["rounds"] == 6


def test_validate_rejects_bad_csr():
    rp = torch.tensor([0, 2, 3, 4], dtype=torch.int64, device="cuda")
    ci = torch.tensor([2, 1, 0, 0], dtype=torch.int32, device="cuda")  # row 0 unsorted
    assert sgr.validate_csr(rp, ci) & 4
    with pytest.raises(RuntimeError, match="invalid"):
        sgr.color(rp, ci, validate=True)
    # unsorted rows are accepted (and colored exactly) with opts->unsorted_rows
    sgr.color(rp, ci, validate=True, unsorted_rows=True)
    g = gen.config(1)
    assert sgr.validate_csr(*dev(g)) == 0


def shuffled_rows(g, seed):
    """Same graph, every row's entries in a random order (the contract's sorted order off)."""
    rng = np.random.default_rng(seed)
    ci = g.col_idx.copy()
    for v in range(g.n):
        a, b = int(g.row_ptr[v]), int(g.row_ptr[v + 1])
        ci[a:b] = rng.permutation(ci[a:b])
    return gen.Graph(g.n, g.nnz, g.row_ptr.copy(), ci, g.name + "-shuffled")


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_unsorted_rows_flag(seed, tb):
    """opts->unsorted_rows: F_1 scans whole rows; colors, R and |W_r| equal the oracle's
    (which never depends on row order) for graphs whose rows are shuffled."""
    g = random_graph(seed, n=300) if seed < 4 else gen.rmat(12, 8, 0.57, 0.19, 0.19, seed=seed)
    h = shuffled_rows(g, seed)
    rp, ci = dev(h)
    ref = oracle.jacobi(h, tb)
    for mode in ("persistent", "host"):
        res = sgr.color(rp, ci, RULE[tb], trace=True, unsorted_rows=True, loop_mode=mode)
        assert res.stats["rounds"] == ref.rounds
        assert np.array_equal(res.colors.cpu().numpy(), ref.colors)
        assert np.array_equal(res.round_sizes, ref.round_sizes)


@pytest.mark.parametrize("B", [64, 96, 128, 256, 384, 512])
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_block_size_never_changes_the_result(B, tb):
    """opts->block_size (the paper's Fig. 8 parameter) is performance only: the
    hub build (R-MAT with multi-chunk rows), the flat build (stencil) and both loop modes
    give the oracle's colors, R and |W_r| at every supported size."""
    for g in (gen.rmat(13, 8, 0.57, 0.19, 0.19, seed=2), gen.stencil3d(12, 11, 10, 27),
              degree_boundary_graph()):
        ref = oracle.jacobi(g, tb)
        rp, ci = dev(g)
        for mode in ("persistent", "host"):
            res = sgr.color(rp, ci, RULE[tb], trace=True, block_size=B, loop_mode=mode)
            assert res.stats["rounds"] == ref.rounds, (g.name, B, mode)
            assert np.array_equal(res.colors.cpu().numpy(), ref.colors), (g.name, B, mode)
            assert np.array_equal(res.round_sizes, ref.round_sizes)
        res = sgr.color(rp, ci, RULE[tb], block_size=B, color_bits=32)
        assert np.array_equal(res.colors.cpu().numpy(), ref.colors), (g.name, B, "int32")


@pytest.mark.parametrize("B", [32, 64, 128, 256, 512, 1024])
def test_block_size_topology_driven_and_steps(B):
    """Per-vertex kernels take any multiple of 32 up to 1024: the topology-driven mapping
    (Algorithm 4, the paper's thread-per-vertex kernel of Fig. 8) and the step entry points."""
    g = gen.rmat(12, 8, 0.57, 0.19, 0.19, seed=3)
    rp, ci = dev(g)
    ref = oracle.jacobi(g, LOW)
    res = sgr.color_topo(rp, ci, "lowid", block_size=B)
    assert np.array_equal(res.colors.cpu().numpy(), ref.colors)
    assert res.stats["rounds"] == ref.rounds
    rng = np.random.default_rng(B)
    snap = rng.integers(0, 9, g.n).astype(np.int32)
    wl = np.sort(rng.choice(g.n, size=g.n // 3, replace=False)).astype(np.int32)
    twl, tsnap = torch.from_numpy(wl).cuda(), torch.from_numpy(snap).cuda()
    tent = sgr.assign(rp, ci, twl, tsnap, block_size=B)
    assert np.array_equal(tent.cpu().numpy(), oracle.assign(g, wl, snap))
    fl = sgr.detect(rp, ci, twl, tsnap, "paper", block_size=B)
    assert np.array_equal(fl.cpu().numpy(), oracle.detect(g, wl, snap, PAP))


def test_block_size_rejected():
    g = gen.rmat(10, 8, 0.57, 0.19, 0.19, seed=1)
    rp, ci = dev(g)
    for B in (33, 16, 2048, 1024):  # 1024 exceeds the fused round kernels' launch bounds
        with pytest.raises(RuntimeError, match="invalid argument"):
            sgr.color(rp, ci, block_size=B)
    with pytest.raises(RuntimeError, match="invalid argument"):
        sgr.color_topo(rp, ci, block_size=48)


def test_color_host_equals_device():
    g = gen.rmat(14, 8, 0.57, 0.19, 0.19, seed=1)
    a = sgr.color(*dev(g)).colors.cpu().numpy()
    rp = torch.from_numpy(g.row_ptr).pin_memory()
    ci = torch.from_numpy(g.col_idx).pin_memory()
    out = torch.zeros(g.n, dtype=torch.int32).pin_memory()
    res = sgr.color_host(rp, ci, out=out)
    assert np.array_equal(out.numpy(), a)
    assert res.stats["rounds"] > 1
    b = sgr.color_host(g.row_ptr, g.col_idx).colors  # pageable numpy also works
    assert np.array_equal(b, a)


@pytest.mark.parametrize("tb", [LOW, PAP])
def test_color_host_batch_pipelined(tb):
    """sgr_color_host_batch: uploads/downloads overlapped with the colorings (two device
    buffer sets, copy streams) give each graph the oracle's coloring — graphs of different
    sizes (the buffer sets are reused across sizes), an empty one, an edgeless one, one
    repeated, pinned torch and pageable numpy inputs mixed."""
    gs = [gen.config(1), random_graph(3, n=300), gen.stencil3d(9, 9, 9), random_graph(5, n=1),
          gen.config(1), degree_boundary_graph()]
    empty = (np.zeros(1, np.int64), np.zeros(0, np.int32))
    edgeless = (np.zeros(6, np.int64), np.zeros(0, np.int32))
    host = []
    for i, g in enumerate(gs):
        if i % 2 == 0:
            host.append((torch.from_numpy(g.row_ptr).pin_memory(), torch.from_numpy(g.col_idx).pin_memory()))
        else:
            host.append((g.row_ptr, g.col_idx))
    host = host[:2] + [empty] + host[2:4] + [edgeless] + host[4:]
    res = sgr.color_host_batch(host, RULE[tb])
    assert len(res) == len(host)
    assert res[2].colors.size == 0
    assert np.array_equal(res[5].colors, np.ones(5, np.int32))
    r = [x for i, x in enumerate(res) if i not in (2, 5)]
    for g, x in zip(gs, r):
        ref = oracle.jacobi(g, tb)
        assert np.array_equal(x.colors, ref.colors), g.name
        assert x.stats["rounds"] == ref.rounds
    assert sgr.color_host_batch([], RULE[tb]) == []


# ----------------------------------------------------------------------------- step API
@pytest.mark.parametrize("seed", range(16))
def test_step_entry_points(seed):
    rng = np.random.default_rng(seed)
    g = random_graph(seed, n=int(rng.integers(1, 400)))
    rp, ci = dev(g)
    snap = rng.integers(0, 9, g.n).astype(np.int32)
    wl = np.sort(rng.choice(g.n, size=int(rng.integers(0, g.n + 1)), replace=False)).astype(np.int32)
    twl = torch.from_numpy(wl).cuda()
    tsnap = torch.from_numpy(snap).cuda()
    tent = sgr.assign(rp, ci, twl, tsnap)
    assert np.array_equal(tent.cpu().numpy(), oracle.assign(g, wl, snap))
    for tb in (LOW, PAP):
        fl = sgr.detect(rp, ci, twl, tsnap, RULE[tb])
        ref = oracle.detect(g, wl, snap, tb)
        assert np.array_equal(fl.cpu().numpy(), ref)
        out = sgr.compact(twl, fl)
        assert np.array_equal(out.cpu().numpy(), wl[ref.astype(bool)])
    colors = tsnap.clone()
    sgr.commit(twl, tent, colors)
    exp = snap.copy()
    exp[wl] = oracle.assign(g, wl, snap)
    assert np.array_equal(colors.cpu().numpy(), exp)


@pytest.mark.parametrize("seed", range(8))
def test_step_assign_with_self_loops(seed):
    """Reading C7 on the step API: sgr_assign is Alg. 5 l.5-6 literally, so a listed
    self-loop forbids v's own snapshot color; GPU and oracle agree on graphs with self-loops
    and duplicate entries under arbitrary snapshots (and detection never flags a loop)."""
    rng = np.random.default_rng(100 + seed)
    h = with_loops_and_dups(random_graph(seed, n=int(rng.integers(2, 300))), seed)
    rp, ci = dev(h)
    snap = rng.integers(0, 7, h.n).astype(np.int32)
    wl = np.arange(h.n, dtype=np.int32)
    twl, tsnap = torch.from_numpy(wl).cuda(), torch.from_numpy(snap).cuda()
    assert np.array_equal(sgr.assign(rp, ci, twl, tsnap).cpu().numpy(), oracle.assign(h, wl, snap))
    for tb in (LOW, PAP):
        assert np.array_equal(sgr.detect(rp, ci, twl, tsnap, RULE[tb]).cpu().numpy(),
                              oracle.detect(h, wl, snap, tb))
    # one vertex with a self-loop, snapshot color 1: l.6 forbids 1, so the first fit is 2
    one = raw_csr(1, [(0, 0)])
    t = sgr.assign(*dev(one), torch.zeros(1, dtype=torch.int32, device="cuda"),
                   torch.ones(1, dtype=torch.int32, device="cuda"))
    assert t.cpu().tolist() == [2]


def test_step_loop_reproduces_algorithm5():
    """Driving assign -> commit -> detect -> compact from Python = the fused library path."""
    g = gen.rmat(13, 8, 0.57, 0.19, 0.19, seed=6)
    rp, ci = dev(g)
    colors = torch.zeros(g.n, dtype=torch.int32, device="cuda")
    wl = torch.arange(g.n, dtype=torch.int32, device="cuda")
    rounds = 0
    while wl.numel():
        rounds += 1
        snapshot = colors.clone()
        tent = sgr.assign(rp, ci, wl, snapshot)
        sgr.commit(wl, tent, colors)
        flags = sgr.detect(rp, ci, wl, colors)
        wl = sgr.compact(wl, flags)
    ref = oracle.jacobi(g, LOW)
    assert rounds == ref.rounds
    assert np.array_equal(colors.cpu().numpy(), ref.colors)
    assert torch.equal(sgr.color(rp, ci).colors, colors)


def test_compact_large_ragged():
    rng = np.random.default_rng(0)
    for L in (1, 1023, 1024, 1025, 300_001):
        wl = rng.integers(0, 1 << 30, L).astype(np.int32)
        fl = (rng.random(L) < 0.37).astype(np.uint8)
        out = sgr.compact(torch.from_numpy(wl).cuda(), torch.from_numpy(fl).cuda())
        assert np.array_equal(out.cpu().numpy(), wl[fl.astype(bool)])


# ----------------------------------------------------------------------------- full size
@pytest.mark.slow
@pytest.mark.parametrize("cfg", [2, 3, 4, 6, 7, 8])
def test_full_size_configs_bit_exact(cfg):
    """BASELINE.json configs 2-4 and the extra workloads 6-8 (Table I shapes, permuted cfg4)
    at full size, in the launch configuration bench.py times
    (default options), against the full oracle (OpenMP over each round's independent
    per-vertex loops; identical to the single-threaded oracle by construction)."""
    g = gen.config(cfg)
    check_full(g, LOW)


@pytest.mark.parametrize("seed", range(16))
@pytest.mark.parametrize("tb", [LOW, PAP])
@pytest.mark.parametrize("mapping", [1, 2])
def test_flat_bin0_mappings_small(seed, tb, mapping):
    """opts->flat_bin0 forces the flat build's bin-0 mapping (1: 4-lane groups, 2: the
    thread-per-vertex instantiation) on small graphs of every family: same result."""
    check_full(random_graph(seed, n=300), tb, flat_bin0=mapping)


@pytest.mark.parametrize("maker", [
    lambda: gen.stencil3d(24, 24, 24, 27),
    lambda: gen.stencil2d(57, 31, 5),
    lambda: gen.er(1 << 15, 8 << 15, seed=3),
    lambda: gen.rmat(14, 10, 0.25, 0.25, 0.25, seed=2),
], ids=["s27-24", "s5", "er15", "rmat-er14"])
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_flat_bin0_thread_families(maker, tb):
    check_full(maker(), tb, flat_bin0=2)


@pytest.mark.parametrize("maker", [
    lambda: gen.stencil3d(24, 24, 24, 27),
    lambda: gen.stencil2d(80, 61, 9),
    lambda: gen.er(1 << 14, 8 << 14, seed=4),
], ids=["s27-24", "s9", "er14"])
@pytest.mark.parametrize("mapping", [1, 2])
@pytest.mark.parametrize("B", [128, 256, 768])
def test_flat_kernels_int32_words_and_block_sizes(maker, mapping, B):
    """The flat build's kernels (dense passes with byte gathers of a word's low byte, both
    bin-0 mappings) with plain int32 color words and other block sizes: same result."""
    g = maker()
    for tb in (LOW, PAP):
        check_full(g, tb, flat_bin0=mapping, color_bits=32, block_size=B)


@pytest.mark.slow
@pytest.mark.parametrize("maker", [
    lambda: gen.er(1 << 22, 8 << 22, seed=5),
    lambda: gen.rmat(22, 6, 0.25, 0.25, 0.25, seed=6),
], ids=["er22", "rmat-er22"])
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_flat_thread_bin0(maker, tb):
    """Non-local rows and n >= 2^22: the flat build's thread-per-vertex instantiation
    (k_persistent<..., T0>) against the oracle, both rules; the host loop (4-lane groups)
    agrees too."""
    g = maker()
    res, _ = check_full(g, tb)
    res_h = sgr.color(*dev(g), RULE[tb], loop_mode="host")
    assert torch.equal(res_h.colors, res.colors)


@pytest.mark.slow
def test_nnz_beyond_2_31_full_size():
    """Row offsets past 2^31 (reading C17): cfg5's shape (R-MAT scale 27) with edge factor 9,
    nnz ~ 2.39e9 > 2^31 (cfg5 itself has 2,125,681,752 entries, just below 2^31), on one GPU
    against the full oracle (OpenMP), element by element (colors, R, |W_r|, sum deg(W_r)),
    plus the partitioned protocol on 2 partitions of the same device. Rows of every degree
    bin, including multi-chunk bin-2 rows, start beyond offset 2^31. Runs in the default
    -m gpu suite (a few minutes: generation and the OpenMP oracle dominate)."""
    g = gen.config(9)
    deg = np.diff(g.row_ptr)
    past = g.row_ptr[:-1] >= 2 ** 31
    assert g.nnz > 2 ** 31 and past.any()
    assert (deg[past] <= 32).any() and ((deg[past] > 32) & (deg[past] <= 256)).any()
    assert (deg[past] > 1020).any()  # multi-chunk rows (bin 2) beyond 2^31
    res, ref = check_full(g, LOW)
    assert res.stats["color_bits"] == 16
    rp, ci = dev(g)
    part = sgr.color_partitioned(rp, ci, 2)
    assert np.array_equal(part.colors.cpu().numpy(), ref.colors)
    assert part.stats["rounds"] == ref.rounds


@pytest.mark.slow
def test_cfg5_full_size():
    """BASELINE config 5 (R-MAT scale 27, ef 8: nnz = 2,125,681,752, int64 offsets) on one
    GPU in bench.py's launch configuration against the full oracle, element by element."""
    g = gen.config(5)
    res, ref = check_full(g, LOW)
    assert res.stats["color_bits"] == 16


# ----------------------------------------------------------------------------- multi-GPU path
@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("tb", [LOW, PAP])
@pytest.mark.parametrize("transport", ["device", "hostloop"])
def test_partitioned_equals_single_gpu(P, tb, transport, monkeypatch):
    """The distributed protocol on P partitions of one device is bit-exact, with both
    transports: the device-side exchange (k_persistent_dist: color words stored into every
    replica, barrier across parts, one cooperative launch) and the host-driven rounds with
    a padded all-gather (pack -> gather -> apply, lockstep advance)."""
    if transport == "hostloop":
        monkeypatch.setenv("SGR_DIST_HOSTLOOP", "1")
    # the 40-plane stencil's slab parts have few boundary vertices: the device exchange
    # then stores each color word only into the replicas that read it (boundary masks)
    for g in (gen.config(1), degree_boundary_graph(), random_graph(7, n=300),
              gen.stencil3d(14, 13, 12, 27), gen.stencil3d(20, 20, 40, 27)):
        rp, ci = dev(g)
        ref = oracle.jacobi(g, tb)
        res = sgr.color_partitioned(rp, ci, P, tiebreak=RULE[tb])
        assert np.array_equal(res.colors.cpu().numpy(), ref.colors), (g.name, P)
        assert res.stats["rounds"] == ref.rounds
        assert res.stats["vertices_processed"] == ref.vertices_processed
        assert res.stats["num_colors"] == ref.num_colors
        if P > 1:
            assert res.stats["transport"] == ("device" if transport == "device" else "allgather")


@pytest.mark.parametrize("P", [1, 3])
def test_partitioned_graph_replay(P, monkeypatch):
    """SGR_DIST_GRAPHS=1: each pass (+ exchange) captured per capacity bucket and replayed;
    the rounds, colors and counts are those of the eager loop and of the oracle (the
    bucketed all-gather capacity pads records, the counts in the payload bound them)."""
    monkeypatch.setenv("SGR_DIST_GRAPHS", "1")
    monkeypatch.setenv("SGR_DIST_HOSTLOOP", "1")
    for g in (gen.config(1), degree_boundary_graph(), gen.stencil3d(12, 12, 12)):
        rp, ci = dev(g)
        for tb in (LOW, PAP):
            ref = oracle.jacobi(g, tb)
            res = sgr.color_partitioned(rp, ci, P, tiebreak=RULE[tb])
            assert np.array_equal(res.colors.cpu().numpy(), ref.colors), (g.name, P, tb)
            assert res.stats["rounds"] == ref.rounds
            assert res.stats["vertices_processed"] == ref.vertices_processed


@pytest.mark.parametrize("P", [1, 3])
@pytest.mark.parametrize("transport", ["device", "hostloop"])
def test_partitioned_color_overflow_rerun(P, transport, monkeypatch):
    """Partitions see a packed overflow in the same exchange and all redo the coloring
    with int32 words (color_cap lowered below K_300's colors by the test hook)."""
    if transport == "hostloop":
        monkeypatch.setenv("SGR_DIST_HOSTLOOP", "1")
    g = degree_boundary_graph()
    rp, ci = dev(g)
    for tb in (LOW, PAP):
        ref = oracle.jacobi(g, tb)
        res = sgr.color_partitioned(rp, ci, P, tiebreak=RULE[tb], color_cap=40)
        assert np.array_equal(res.colors.cpu().numpy(), ref.colors), (P, tb)
        assert res.stats["color_bits"] == 32
        assert res.stats["rounds"] == ref.rounds


@pytest.mark.parametrize("bits", [16, 32])
def test_partitioned_random_ranges_and_widths(bits):
    g = gen.rmat(14, 8, 0.57, 0.19, 0.19, seed=3)
    rp, ci = dev(g)
    ref = sgr.color(rp, ci).colors
    rng = np.random.default_rng(0)
    for P in (2, 4, 7):
        cuts = np.sort(rng.integers(0, g.n + 1, P - 1))
        ranges = np.concatenate([[0], cuts, [g.n]]).astype(np.int64)
        res = sgr.color_partitioned(rp, ci, P, ranges=ranges, color_bits=bits)
        assert torch.equal(res.colors, ref), (P, ranges)


@pytest.mark.parametrize("transport", ["device", "nccl"])
def test_nccl_world1_color_dist(transport, monkeypatch):
    """sgr_comm_init + sgr_color_dist over a one-rank NCCL communicator (the box has one
    GPU; multi-rank NCCL is exercised by bench.py under torchrun on a multi-GPU node)."""
    import socket

    import torch.distributed as dist
    from paper_conf_ipps_licqfsty16_b200.dist import Comm, color_dist
    if transport == "nccl":
        monkeypatch.setenv("SGR_DIST_TRANSPORT", "nccl")
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0,
                            world_size=1, device_id=torch.device("cuda", 0))
    try:
        comm = Comm(0, 1, 0)
        for g in (gen.config(1), degree_boundary_graph()):
            rp, ci = dev(g)
            res = color_dist(comm, rp, ci, g.n, 0, g.n)
            ref = oracle.jacobi(g, LOW)
            assert np.array_equal(res.colors.cpu().numpy(), ref.colors)
            assert res.stats["rounds"] == ref.rounds
        comm.close()
    finally:
        dist.destroy_process_group()


# ------------------------------------------- topology-driven mapping (Algorithm 4, T-base)
def check_topo(g, tb):
    rp, ci = dev(g)
    res = sgr.color_topo(rp, ci, RULE[tb], trace=True)
    ref = oracle.jacobi(g, tb, nthreads=oracle.max_threads())
    assert res.stats["rounds"] == ref.rounds, (g.name, res.stats["rounds"], ref.rounds)
    assert np.array_equal(res.colors.cpu().numpy(), ref.colors), g.name
    assert np.array_equal(res.round_sizes, ref.round_sizes), g.name
    assert res.stats["num_colors"] == ref.num_colors
    assert res.stats["vertices_processed"] == ref.vertices_processed
    assert res.stats["edges_scanned"] == ref.edges_scanned
    return res


@pytest.mark.parametrize("seed", range(24))
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_topology_driven_random_graphs(seed, tb):
    check_topo(random_graph(seed), tb)


@pytest.mark.parametrize("maker", [
    lambda: gen.config(1),
    lambda: gen.stencil3d(20, 20, 20, 27),
    lambda: gen.er(1 << 14, 8 << 14, seed=5),
    lambda: gen.rmat(14, 10, 0.45, 0.15, 0.15, seed=2),
], ids=["cfg1", "s27-20", "er14", "rmat-g14"])
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_topology_driven_families(maker, tb):
    check_topo(maker(), tb)


def test_topology_driven_equals_data_driven_and_edge_cases():
    g = gen.rmat(16, 8, 0.57, 0.19, 0.19, seed=9)
    rp, ci = dev(g)
    a = sgr.color(rp, ci).colors
    b = sgr.color_topo(rp, ci).colors
    assert torch.equal(a, b)
    # self-loops and duplicates (readings C7, C9), n = 1 with a loop, nnz = 0
    r2 = raw_csr(4, [(0, 0), (0, 1), (0, 1), (1, 0), (1, 2), (2, 1), (2, 3), (3, 2), (3, 3)])
    res = check_topo(r2, LOW)
    assert res.stats["rounds"] >= 1
    z = gen.from_edges(5, np.zeros((0, 2), np.int64))
    res = sgr.color_topo(*dev(z))
    assert res.colors.cpu().tolist() == [1] * 5 and res.stats["rounds"] == 1


# --------------------------------- list maintenance of high-degree rows (lazy / kept lists)
@pytest.mark.parametrize("maker", [
    lambda: gen.rmat(16, 16, 0.60, 0.15, 0.15, seed=11),     # hubs of several 1020-entry chunks
    lambda: gen.rmat(17, 8, 0.57, 0.19, 0.19, seed=12),
    lambda: gen.rmat(15, 12, 0.57, 0.19, 0.19, seed=13, permute=True),
], ids=["rmat16-ef16", "rmat17", "rmat15-perm"])
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_multi_chunk_hub_lists(maker, tb):
    """Graphs whose hubs span several chunks and lose neighbours at different rounds: the
    kept / compacted list transitions, single-chunk lazy rewrites and the finalize skip must
    all reproduce the oracle's colors, rounds and per-round worklist sizes."""
    g = maker()
    deg = np.diff(g.row_ptr)
    assert deg.max() > 2 * 1020, deg.max()  # really multi-chunk
    res, _ = check_full(g, tb)
    assert res.stats["entries_read"] <= res.stats["edges_scanned"]


def hub_core_graph(seed, hubs, hub_deg, n):
    """A clique of `hubs` hub vertices, each adjacent to `hub_deg` random other vertices,
    which also form a sparse random graph among themselves: the hubs see every small color
    and conflict with each other for many rounds (the early-exit case of bin 2)."""
    rng = np.random.default_rng(seed)
    hub_ids = rng.choice(n, hubs, replace=False)
    iu = np.triu_indices(hubs, 1)
    core = np.stack([hub_ids[iu[0]], hub_ids[iu[1]]], 1)
    spokes = np.stack([np.repeat(hub_ids, hub_deg), rng.integers(0, n, hubs * hub_deg)], 1)
    rest = rng.integers(0, n, size=(4 * n, 2))
    return gen.from_edges(n, np.concatenate([core, spokes, rest]).astype(np.int64))


@pytest.mark.parametrize("hub_deg", [300, 900, 5000], ids=["one-batch+", "single-chunk", "multi-chunk"])
@pytest.mark.parametrize("tb", [LOW, PAP])
@pytest.mark.parametrize("seed", [0, 1])
def test_bin2_early_exit(hub_deg, tb, seed):
    """A clique of hubs whose rows span one batch, one chunk or several chunks, seeing every
    small color: the trimmed bin-2 lists, the finalize merge and (in SGR_EARLY builds) the
    chunk early exit — stop once the vertex conflicts and colors 1..k are all forbidden, the
    unread entries staying listed — keep colors, R, |W_r| and sum deg(W_r) bit-exact, with
    fewer entries read than the untrimmed rounds scan."""
    g = hub_core_graph(seed, 48, hub_deg, 20000)
    res, _ = check_full(g, tb)
    assert res.stats["entries_read"] < res.stats["edges_scanned"]


# ----------------------------------------------------------------------------- §8(f) item 4
def check_gs(g, K, part, tb):
    rp, ci = dev(g)
    res = sgr.color_gs(rp, ci, K, part, RULE[tb], trace=True)
    ref = oracle.gauss_seidel(g, K, part, tb)
    assert res.stats["rounds"] == ref.rounds, (g.name, K, part, res.stats["rounds"], ref.rounds)
    assert np.array_equal(res.colors.cpu().numpy(), ref.colors), (g.name, K, part)
    assert np.array_equal(res.round_sizes, ref.round_sizes)
    assert np.array_equal(res.round_edges, ref.trace["w_edges"])
    assert res.stats["num_colors"] == ref.num_colors
    return res, ref


@pytest.mark.parametrize("seed", range(16))
@pytest.mark.parametrize("part", ["strided", "blocked"])
def test_gs_substeps_random_graphs(seed, part):
    """K-sub-step Gauss-Seidel rounds against the oracle's O3:
    bit-exact colors, R, |W_r| and sum deg(W_r), both rules, K in 1..16."""
    g = random_graph(seed, n=200)
    for K in (1, 2, 3, 16):
        for tb in (LOW, PAP):
            check_gs(g, K, 0 if part == "strided" else 1, tb)


@pytest.mark.parametrize("maker", [
    lambda: gen.config(1),
    lambda: gen.stencil3d(16, 15, 14, 27),
    lambda: gen.er(1 << 14, 8 << 14, seed=5),
    lambda: gen.rmat(13, 10, 0.45, 0.15, 0.15, seed=3),
], ids=["cfg1", "s27", "er14", "rmat-g13"])
@pytest.mark.parametrize("K", [4, 16, 64])
def test_gs_substeps_families(maker, K):
    g = maker()
    for part in (0, 1):
        check_gs(g, K, part, LOW)


def test_gs_one_substep_equals_jacobi_and_loops():
    g = gen.config(1)
    rp, ci = dev(g)
    a = sgr.color_gs(rp, ci, 1, "strided").colors
    assert torch.equal(a, sgr.color(rp, ci).colors)
    h = with_loops_and_dups(random_graph(3, n=150), 3)  # listed self-loops: Alg. 5 l.5-6 literally
    for K in (1, 4):
        check_gs(h, K, 0, LOW)


@pytest.mark.parametrize("tb", [LOW, PAP])
def test_gs_inplace_nondeterministic_is_proper(tb):
    """Partition 2: the paper's in-place assignment (nondeterministic): every run ends with a
    proper coloring, colors in [1, deg + 1], and W shrinking every round."""
    for g in (gen.config(1), gen.stencil3d(20, 20, 20, 27), random_graph(7, n=300)):
        rp, ci = dev(g)
        deg = np.diff(g.row_ptr)
        for _ in range(3):
            res = sgr.color_gs(rp, ci, 1, "inplace", RULE[tb], trace=True)
            c = res.colors.cpu().numpy()
            assert c.min() >= 1 and np.all(c <= deg + 1)
            src = np.repeat(np.arange(g.n), deg)
            assert not np.any((c[src] == c[g.col_idx]) & (src != g.col_idx)), g.name
            assert np.all(np.diff(res.round_sizes) < 0)


@pytest.mark.slow
@pytest.mark.parametrize("cfg", [3, 4])
def test_gs_full_size(cfg):
    """cfg3 / cfg4 at full size with K = 16 strided sub-steps against the oracle's O3."""
    check_gs(gen.config(cfg), 16, 0, LOW)


# ----------------------------------------------------------------------------- dense passes
def local_long_rows(nx, ny, every=997, width=120):
    """A 9-point grid plus, every `every` vertices, edges to the next `width` ids: rows of
    33..256 entries (bin 1) that stay local in id space, so the flat build's dense passes
    take their long-row path."""
    g = gen.stencil2d(nx, ny, 9)
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    e = [np.stack([src, g.col_idx], 1)]
    for v in range(0, g.n - width - 1, every):
        e.append(np.stack([np.full(width, v), np.arange(v + 1, v + 1 + width)], 1))
    return gen.from_edges(g.n, np.concatenate(e).astype(np.int64))


def far_edges(N=40, gap=33000, every=3001):
    """A 27-point stencil plus a few edges v -- v + gap with gap > 2^15 - 1: still local on
    average (dense passes run) but some w - v does not fit the dense passes' 16-bit deltas
    (dcol), so they must fall back to staging col_idx."""
    g = gen.stencil3d(N, N, N, 27)
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    extra = np.array([[v, v + gap] for v in range(0, g.n - gap, every)], np.int64)
    return gen.from_edges(g.n, np.concatenate([np.stack([src, g.col_idx], 1), extra]))


@pytest.mark.parametrize("maker", [
    lambda: gen.stencil3d(40, 40, 40, 27),
    lambda: gen.stencil3d(37, 35, 33, 7),
    lambda: gen.stencil2d(401, 299, 5),
    lambda: gen.stencil2d(250, 250, 9),
    lambda: local_long_rows(300, 301),
    lambda: far_edges(),
], ids=["s27-40", "s7-odd", "s5-odd", "s9-250", "long-rows", "far-edges"])
@pytest.mark.parametrize("tb", [LOW, PAP])
def test_dense_passes_of_the_flat_build(maker, tb):
    """Graphs with local rows (mean row width < n/16) run their first rounds as dense passes
    (bitmap worklists, thread per vertex, staged rows) and switch to sparse passes through
    the bitmap -> worklist compaction: colors, R, |W_r| and sum deg(W_r) equal the oracle's,
    in both color widths, and equal the host loop (which never uses dense passes)."""
    g = maker()
    rp, ci = dev(g)
    ref = oracle.jacobi(g, tb)
    for bits in (16, 32):
        res, _ = check_full(g, tb, color_bits=bits)
        host = sgr.color(rp, ci, RULE[tb], loop_mode="host", color_bits=bits)
        assert torch.equal(res.colors, host.colors)
    for B in (64, 192, 512):
        res = sgr.color(rp, ci, RULE[tb], block_size=B)
        assert np.array_equal(res.colors.cpu().numpy(), ref.colors), B
