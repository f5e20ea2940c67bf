"""bench.py's multi-GPU leg (torchrun, one process per GPU, NCCL over NVLink).

Every rank generates the same seeded graph (the generator is deterministic), takes its
nnz-balanced contiguous vertex range (sgr_partition), uploads its owned rows with global
column ids, and runs sgr_color_dist — one fused pass + one NCCL all-gather of recolored
vertices per round, inside libsgr. Timing: barrier + synchronize on both sides of K steps,
CUDA events on the launching stream, MAX over ranks (all_reduce). Strong scaling: the total
work (the graph) is fixed as N grows.
"""
from __future__ import annotations

import json
import os
import statistics
import time

import numpy as np


def rank_env():
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def owned_rows(row_ptr: np.ndarray, col_idx: np.ndarray, rank: int, world: int):
    """(v_begin, v_end, local_row_ptr, local_col_idx) of this rank's nnz-balanced range."""
    import paper_conf_ipps_licqfsty16_b200 as sgr
    from .dist import local_rows
    ranges = sgr.partition(row_ptr, world)
    lo, hi = int(ranges[rank]), int(ranges[rank + 1])
    lrp, lci = local_rows(row_ptr, col_idx, lo, hi)
    return lo, hi, lrp, np.ascontiguousarray(lci), ranges


def run(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_licqfsty16_b200 as sgr
    from paper_conf_ipps_licqfsty16_b200 import gen
    from .dist import Comm, color_dist

    rank, world, local = rank_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    g = gen.config(args.config)
    lo, hi, lrp, lci, ranges = owned_rows(g.row_ptr, g.col_idx, rank, world)
    rp_d = torch.from_numpy(lrp).to(dev)
    ci_d = torch.from_numpy(lci).to(dev) if len(lci) else torch.zeros(4, dtype=torch.int32, device=dev)
    comm = Comm(rank, world, local)
    stream = torch.cuda.current_stream()

    def step():
        return color_dist(comm, rp_d, ci_d, g.n, lo, hi, args.tiebreak)

    for _ in range(max(args.warmup, 3)):
        res = step()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    dist.barrier()
    torch.cuda.synchronize()
    for i in range(args.steps):
        ev[i][0].record(stream)
        res = step()
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    dist.barrier()
    ms = statistics.mean(a.elapsed_time(b) for a, b in ev)
    t = torch.tensor([ms], device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    # every replica holds the full coloring: check ranks agree
    h = torch.tensor([int(res.colors.sum().item()), res.stats["rounds"]], device=dev, dtype=torch.int64)
    hs = [torch.zeros_like(h) for _ in range(world)]
    dist.all_gather(hs, h)
    agree = all(torch.equal(hs[0], x) for x in hs)
    if rank == 0:
        line = {"metric": "coloring GTEPS at 1/2/4/8 B200 (% HBM roofline); colors used vs seq greedy",
                "value": g.nnz / (ms_max * 1e-3) / 1e9, "unit": "GTEPS", "n_gpus": world,
                "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": ms_max,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
                "dtype": "int32", "data": "synthetic",
                "config": {"workload": gen.CONFIG_NAMES[args.config], "n": g.n, "nnz": g.nnz,
                           "tiebreak": args.tiebreak,
                           "parallelism": f"{world} contiguous nnz-balanced vertex ranges, "
                                          "NCCL all-gather of recolored vertices per round",
                           "ranges": [int(x) for x in ranges]},
                "rounds": res.stats["rounds"], "num_colors": res.stats["num_colors"],
                "replicas_agree": agree, "gpu_launches": res.stats["launches"] * args.steps}
        print(json.dumps(line), flush=True)
    comm.close()
    dist.destroy_process_group()
