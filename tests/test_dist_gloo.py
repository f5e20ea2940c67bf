"""Multi-process (world size 2, gloo, CPU) tests of the distributed path's host logic.

What runs on each rank is what bench.py's N>1 leg and sgr_color_dist do around the GPU
kernels: the nnz-balanced partition (libsgr's sgr_partition, host code), slicing of owned
rows with global column ids (benchdist.owned_rows), and the per-round exchange protocol —
records (v, new color) of the rank's part of W_{k+1}, a PADDED all-gather whose capacity is
the previous round's largest count (valid because W only shrinks), counts in the header,
termination when the gathered counts sum to zero. The per-vertex arithmetic of a round is
done here by the CPU oracle's step functions (test infrastructure), so the test pins the
protocol against the single-process oracle on CPU.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_ipps_licqfsty16_b200 import benchdist, gen


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _fused_round_protocol(rank, world, g, tb):
    """Jacobi SGR where this rank computes only its owned vertices (fused pass: detect of
    round k + assign of round k+1 against the replica snapshot) and learns the others'
    recolored vertices through the padded all-gather."""
    lo, hi, lrp, lci, ranges = benchdist.owned_rows(g.row_ptr, g.col_idx, rank, world)
    # owned rows really are the global rows, with global ids
    assert np.array_equal(lci, g.col_idx[g.row_ptr[lo]:g.row_ptr[hi]])
    assert lrp[0] == 0 and lrp[-1] == g.row_ptr[hi] - g.row_ptr[lo]
    n = g.n
    replica = np.ones(n, np.int32)  # C_1: every vertex took color 1
    # F_1 (no gathers): owned v in W_2 iff it loses to a neighbour (all colors are 1)
    own = np.arange(lo, hi, dtype=np.int32)
    fl = oracle.detect(g, own, replica, tb) if len(own) else np.zeros(0, np.uint8)
    W = own[fl.astype(bool)]
    new_colors = np.full(len(W), 2, np.int32)
    cap = hi - lo  # first exchange: the owner's range bounds its count
    caps = torch.zeros(world, dtype=torch.int64)
    dist.all_gather(list(caps.chunk(world)), torch.tensor([cap], dtype=torch.int64))
    cap = int(caps.max())
    rounds = 1
    while True:
        # ---- exchange W_{k+1} records: [count, v0, c0, v1, c1, ...] padded to cap
        send = torch.zeros(1 + 2 * cap, dtype=torch.int64)
        send[0] = len(W)
        assert len(W) <= cap
        send[1:1 + 2 * len(W):2] = torch.from_numpy(W.astype(np.int64))
        send[2:2 + 2 * len(W):2] = torch.from_numpy(new_colors.astype(np.int64))
        recv = [torch.zeros_like(send) for _ in range(world)]
        dist.all_gather(recv, send)
        counts = [int(r[0]) for r in recv]
        for q, r in enumerate(recv):  # every record lands in every replica (incl. own)
            c = counts[q]
            vs = r[1:1 + 2 * c:2].numpy()
            cs = r[2:2 + 2 * c:2].numpy()
            replica[vs] = cs
        if sum(counts) == 0:
            break
        rounds += 1
        cap = max(counts)  # W only shrinks: a valid capacity for the next exchange
        # ---- fused pass F_k over the owned worklist W against the snapshot `replica`
        if len(W):
            conflict = oracle.detect(g, W, replica, tb).astype(bool)
            tent = oracle.assign(g, W, replica)
            W, new_colors = W[conflict], tent[conflict]
        else:
            new_colors = np.zeros(0, np.int32)
    return replica, rounds


def _worker(rank, world, port, results, cfg, tb):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = gen.rmat(12, 8, 0.57, 0.19, 0.19, seed=5) if cfg == "rmat12" else gen.config(1)
        colors, rounds = _fused_round_protocol(rank, world, g, tb)
        results[rank] = (colors.tolist(), rounds)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("cfg,tb", [("rmat12", 0), ("rmat12", 1), ("cfg1", 0)])
def test_gloo_world2_protocol_matches_oracle(cfg, tb):
    world = 2
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), results, cfg, tb), nprocs=world, join=True)
    g = gen.rmat(12, 8, 0.57, 0.19, 0.19, seed=5) if cfg == "rmat12" else gen.config(1)
    ref = oracle.jacobi(g, tb)
    for r in range(world):
        colors, rounds = results[r]
        assert colors == ref.colors.tolist()  # every replica ends with the full coloring
        assert rounds == ref.rounds


def test_owned_rows_cover_the_graph():
    g = gen.config(1)
    parts = [benchdist.owned_rows(g.row_ptr, g.col_idx, r, 4) for r in range(4)]
    assert parts[0][0] == 0 and parts[-1][1] == g.n
    for (lo, hi, lrp, lci, _), nxt in zip(parts, parts[1:] + [None]):
        if nxt is not None:
            assert hi == nxt[0]
        assert len(lci) == lrp[-1]
    nnzs = [len(p[3]) for p in parts]
    assert sum(nnzs) == g.nnz
    assert max(nnzs) - min(nnzs) <= g.degrees.max()  # nnz-balanced up to one row
