#!/usr/bin/env python3
"""Benchmark: deterministic Jacobi-SGR coloring GTEPS on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 4] [--impl ours|reference]

One "step" = one complete coloring (every round of the hot path: F_1, then fused
assign/detect/compact passes until the worklist is empty) of the config's graph, resident in
HBM. GTEPS = input nnz / step time; redundant rounds never inflate it.
Rank 0 prints ONE JSON line. For N > 1 (torchrun) the graph is partitioned into nnz-balanced
contiguous vertex ranges and colored by sgr_color_dist (NCCL exchange per round; strong
scaling: the total work is fixed).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "coloring GTEPS at 1/2/4/8 B200 (% HBM roofline); colors used vs seq greedy"
L2_BYTES = 126 * 1024 * 1024


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=4,
                    help="BASELINE.json config (1-based); 6-8: extra workloads (gen.config)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--tiebreak", default="lowid", choices=["lowid", "paper"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--loop-mode", default="auto")
    ap.add_argument("--dist", action="store_true",
                    help="use the multi-GPU (NCCL) path even for one rank")
    ap.add_argument("--block-size", type=int, default=0,
                    help="threads per block (opts->block_size; 0 = 256)")
    ap.add_argument("--no-secondary", action="store_true",
                    help="skip the secondary paper-rule (v < w) line")
    return ap.parse_args()


# Scattered color-gather ceiling of one B200 (tools/gather_bench.cu: random 4-byte gathers
# into a 64 MB L2-resident array, ~1 distinct 128-byte line per SM-cycle; see
# profiles/r01_ncu_summary.md). The round kernel's binding resource besides HBM.
GATHER_PEAK_G = 271.0


def ncu_metric(workload: str, kernel: str, key: str):
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    return d.get(workload, {}).get(kernel, {}).get(key)


def ncu_traffic(workload: str, kernel: str):
    """DRAM bytes per launch of `kernel` from the committed ncu --set full capture
    (profiles/ncu_traffic.json, written from `ncu -i ... --page raw`), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    e = d.get(workload, {}).get(kernel)
    return None if e is None else int(e["dram_read_bytes"] + e["dram_write_bytes"])


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, gpu_index: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={gpu_index}", f"--query-gpu={q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except FileNotFoundError:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.p.kill()
        self.f.seek(0)
        rows = [r.split(",") for r in self.f.read().strip().splitlines() if r.strip()]
        os.unlink(self.f.name)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            try:
                sm.append(float(r[1]))
                mx = float(r[2])
                for nm, val in zip(names, r[5:9]):
                    if val.strip() == "Active":
                        reasons.add(nm)
            except (ValueError, IndexError):
                continue
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def host_graph(cfg: int):
    from paper_conf_ipps_licqfsty16_b200 import gen
    t0 = time.time()
    g = gen.config(cfg)
    return g, time.time() - t0


def workload_name(cfg):
    from paper_conf_ipps_licqfsty16_b200 import gen
    return gen.CONFIG_NAMES[cfg]


def bench_config(args, g) -> dict:
    """The workload a line is quoted on; identical for our arm and the reference arm."""
    return {"workload": workload_name(args.config), "n": g.n, "nnz": g.nnz,
            "tiebreak": args.tiebreak, "parallelism": "single GPU",
            "l2": "flushed between steps (256 MiB write, outside the step events); "
                  "CSR inputs 1.2 GB > L2",
            "loop_mode": args.loop_mode, "block_size": args.block_size or 256}


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


# The paper's own headline numbers (PAPER.md:5 abstract, :257 Fig. 7; NVIDIA K20c):
# context for the speedup lines, never a target of this metric (different GPU, datasets).
PAPER_CONTEXT = {"speedup_vs_sequential": 3.0, "speedup_vs_csrcolor": 1.5, "gpu": "NVIDIA K20c",
                 "source": "PAPER.md:5 (abstract), :257 (Fig. 7: data-driven 1.5x csrcolor)",
                 "note": "context only: other hardware and datasets (UF matrices, P:234)"}


# ------------------------------------------------------------------------ CPU oracle legs
def oracle_run(g, tiebreak: int, edges_total: int | None, budget_s: float = 30.0):
    """Time the oracle (as it stands) on the box's host cores. A full O2 run if it fits the
    budget; else the first rounds, extrapolated by scanned CSR entries (the unit of work)."""
    import oracle
    cores = oracle.max_threads()
    t0 = time.perf_counter()
    probe = oracle.jacobi(g, tiebreak, nthreads=cores, max_rounds=4)
    t_probe = time.perf_counter() - t0
    if probe.converged:
        return {"seconds": t_probe, "cores": cores, "sample": "full run", "result": probe}
    total = edges_total
    est = None if not total else t_probe * total / max(probe.edges_scanned, 1)
    # total unknown (reference arm, first step): run it in full once to learn it
    if est is None or est <= budget_s:
        t0 = time.perf_counter()
        full = oracle.jacobi(g, tiebreak, nthreads=cores)
        return {"seconds": time.perf_counter() - t0, "cores": cores, "sample": "full run",
                "result": full}
    return {"seconds": est if est is not None else float("nan"), "cores": cores,
            "sample": (f"first {probe.rounds} Jacobi rounds ({probe.edges_scanned} of {total} "
                       f"scanned CSR entries), time extrapolated by scanned entries"),
            "result": None}


def oracle_parity(g, colors, rounds, tiebreak) -> bool:
    """Rank 0 of the multi-GPU line: the replica's colors and R equal the oracle's (O2)."""
    import oracle
    ref = oracle.jacobi(g, 0 if tiebreak == "lowid" else 1, nthreads=oracle.max_threads())
    return bool(np.array_equal(ref.colors, colors)) and ref.rounds == rounds


def alg1_run(g):
    import oracle
    t0 = time.perf_counter()
    c = oracle.alg1(g)
    return int(c.max()), time.perf_counter() - t0


# ------------------------------------------------------------------------ reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    tb = 0 if args.tiebreak == "lowid" else 1
    g, _ = host_graph(args.config)
    cores = oracle.max_threads()
    times = []
    edges_total = None
    res = None
    for i in range(args.warmup + args.steps):
        r = oracle_run(g, tb, edges_total, budget_s=60.0)
        if r["result"] is not None:
            res = r["result"]
            edges_total = res.edges_scanned
        if i >= args.warmup:
            times.append(r["seconds"])
        if r["sample"] != "full run" and i + 1 >= args.warmup + 1:
            break  # sampled: one timed sample is enough
    t = statistics.mean(times)
    value = g.nnz / t / 1e9
    sample = "full oracle run per step" if res is not None else r["sample"]
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "GTEPS",
            "n_gpus": args.gpus, "device": "host cpu", "steps": len(times), "warmup": args.warmup, "ms_per_step": t * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "int32", "data": "synthetic",
            "config": bench_config(args, g),
            "cpu_baseline": {"value": value, "unit": "GTEPS", "cores": cores, "kind": "oracle",
                             "sample": sample, "cpu_model": cpu_model()},
            "e2e": {"value": value, "unit": "GTEPS", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    if res is not None:
        line["rounds"] = res.rounds
        line["num_colors"] = res.num_colors
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------ our arm, 1 GPU
def run_single(args):
    import torch
    import paper_conf_ipps_licqfsty16_b200 as sgr

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    g, gen_s = host_graph(args.config)
    rp_h = torch.from_numpy(g.row_ptr).pin_memory()
    ci_h = torch.from_numpy(g.col_idx).pin_memory()
    rp = rp_h.to(dev, non_blocking=True)
    ci = ci_h.to(dev, non_blocking=True)
    colors = torch.empty(g.n, dtype=torch.int32, device=dev)
    ws = torch.empty(sgr.workspace_bytes(g.n, g.nnz), dtype=torch.uint8, device=dev)
    flush = torch.empty(2 * L2_BYTES // 4, dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream()
    torch.cuda.synchronize()

    colors_sec = torch.empty(g.n, dtype=torch.int32, device=dev)  # secondary-rule output

    def step(profile=False, tiebreak=None):
        return sgr.color(rp, ci, tiebreak or args.tiebreak,
                         out=colors_sec if tiebreak else colors, workspace=ws,
                         profile=profile, loop_mode=args.loop_mode, block_size=args.block_size)

    for _ in range(max(args.warmup, 3)):
        res = step()
    torch.cuda.synchronize()
    # |W_2| (F_1's output) from one traced coloring: the pushes of the round kernel are
    # sum_{k>=2} |W_{k+1}| = sum_{k>=2} |W_k| - |W_2| (the result is deterministic)
    tr = sgr.color(rp, ci, args.tiebreak, trace=True, loop_mode=args.loop_mode,
                   block_size=args.block_size)
    w2 = int(tr.round_sizes[1]) if len(tr.round_sizes) > 1 else 0
    del tr
    torch.cuda.synchronize()

    # timed region: K complete colorings, L2 flushed between them (outside the step events).
    # profile=True records CUDA events around each kernel launch on the launching stream
    # (the persistent round kernel is ONE launch per coloring, so this costs nothing).
    clocks = Clocks(0)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    launches = 0
    kms, kl, kb = {}, {}, {}
    torch.cuda.synchronize()
    wall0 = time.perf_counter()
    for i in range(args.steps):
        flush.fill_(i)
        ev[i][0].record(stream)
        res = step(profile=True)
        ev[i][1].record(stream)
        launches += res.stats["launches"]
        for k, v in res.stats["kernel_ms"].items():
            kms[k] = kms.get(k, 0.0) + v
            kl[k] = kl.get(k, 0) + res.stats["kernel_launches"][k]
            kb[k] = kb.get(k, 0) + res.stats["kernel_bytes"][k]
    torch.cuda.synchronize()
    wall = time.perf_counter() - wall0
    clk = clocks.stop()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    ms = statistics.mean(step_ms)
    st = res.stats
    value = g.nnz / (ms * 1e-3) / 1e9

    peak, peak_src = peaks()
    dom = max(kms, key=lambda k: kms[k])
    total_kernel_ms = sum(kms.values())
    launches_dom = max(kl[dom], 1)
    launch_s = kms[dom] * 1e-3 / launches_dom  # average launch duration (CUDA events)
    # SURVEY §8(d) algorithmic bytes of the fused round kernel (one launch per coloring in
    # the persistent mode), from the method's own counts, independent of trimming:
    #   per scanned edge of rounds >= 2 (sum_k |adj(W_k)|): 4 B col_idx + one color word
    #   per worklist vertex of rounds >= 2 (sum_k |W_k|): 4 B id + 16 B int64 row pair + X[v] + Y[v]
    #   per push (sum_{k>=2} |W_{k+1}|): 4 B
    cb = 2 if st["color_bits"] == 16 else 4
    e_k = st["edges_scanned"] - g.nnz
    v_k = st["vertices_processed"] - g.n
    pushes = max(v_k - w2, 0)
    alg8d = (4 + cb) * e_k + (4 + 16 + 2 * cb) * v_k + 4 * pushes
    # e_k, v_k, pushes are per coloring (one step); kb[dom] sums the K timed steps
    per_launch = (alg8d / (launches_dom / args.steps) if dom == "round"
                  else kb[dom] / launches_dom)
    achieved = per_launch / launch_s / 1e9 if launch_s > 0 else 0.0
    traffic = ncu_traffic(workload_name(args.config), dom)
    roofline = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak,
                "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic,
                "byte_model": "SURVEY.md §8(d): (4+cb)*sum|adj(W_k)| + (20+2cb)*sum|W_k| + 4*pushes, "
                              "k >= 2, cb = color word bytes",
                "peak_source": peak_src,
                "launches_per_step": kl[dom] / args.steps,
                "algorithmic_bytes_per_launch": per_launch,
                "sum_adj_W_k": e_k, "sum_W_k": v_k, "pushes": pushes,
                "dram_frac": (traffic / launch_s / 1e9 / peak) if (traffic and launch_s > 0) else None,
                "lts_read_sectors": ncu_metric(workload_name(args.config), dom, "lts_read_sectors"),
                "trimmed_model": {"bytes_per_launch": kb[dom] / launches_dom,
                                  "achieved": kb[dom] / launches_dom / launch_s / 1e9 if launch_s > 0 else 0.0,
                                  "note": "bytes the trimmed lists actually move (DESIGN.md §5)"},
                "avg_launch_us": kms[dom] * 1e3 / launches_dom,
                "share_of_kernel_time": kms[dom] / total_kernel_ms if total_kernel_ms else None,
                "kernel_ms_per_step": {k: v / args.steps for k, v in kms.items()},
                "whole_step": {"algorithmic_GBps": st["bytes_algorithmic"] / (ms * 1e-3) / 1e9,
                               "frac": st["bytes_algorithmic"] / (ms * 1e-3) / 1e9 / peak},
                "bin_edges": st["bin_edges"], "bin_vertices": st["bin_vertices"],
                "chunk_items": st["chunk_items"], "grid_blocks": st["grid_blocks"],
                "entries_read_per_nnz": st["entries_read"] / g.nnz,
                "entries_written_per_nnz": st["entries_written"] / g.nnz,
                "color_bits": st["color_bits"]}
    # the same kernel against the scattered-gather ceiling (one color gather per entry read)
    g_rate = st["entries_read"] / (kms["round"] / args.steps * 1e-3) / 1e9 if kms.get("round") else 0.0
    roofline["gather"] = {"achieved": g_rate, "peak": GATHER_PEAK_G, "unit": "G gathers/s",
                          "frac": g_rate / GATHER_PEAK_G,
                          "peak_source": "measured, tools/gather_bench.cu (profiles/r01_ncu_summary.md)"}

    # e2e: the same coloring through sgr_color_host from pinned host buffers
    e2e = None
    if not args.no_e2e:
        out_h = torch.empty(g.n, dtype=torch.int32).pin_memory()
        sgr.color_host(rp_h, ci_h, args.tiebreak, out=out_h)
        e_ms = []
        for i in range(min(args.steps, 5)):
            flush.fill_(i)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            sgr.color_host(rp_h, ci_h, args.tiebreak, out=out_h)
            e_ms.append((time.perf_counter() - t0) * 1e3)
        assert torch.equal(out_h, colors.cpu()), "e2e colors differ from device-resident run"
        serial = {"value": g.nnz / (statistics.mean(e_ms) * 1e-3) / 1e9,
                  "ms_per_step": statistics.mean(e_ms), "api": "sgr_color_host, one call per step"}
        # pipelined: the K steps as one sgr_color_host_batch call over K host graphs (the
        # same pinned CSR each step): step i+1's upload and step i-1's download overlap step
        # i's coloring; every step still copies its full inputs and reads its colors back
        K = args.steps
        outs = [torch.empty(g.n, dtype=torch.int32).pin_memory() for _ in range(K)]
        sgr.color_host_batch([(rp_h, ci_h)] * 2, args.tiebreak, outs=outs[:2])  # warm-up
        flush.fill_(7)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        sgr.color_host_batch([(rp_h, ci_h)] * K, args.tiebreak, outs=outs)
        p_ms = (time.perf_counter() - t0) * 1e3 / K
        ref_c = colors.cpu()
        assert all(torch.equal(o, ref_c) for o in outs), "pipelined e2e colors differ"
        e2e = {"value": g.nnz / (p_ms * 1e-3) / 1e9, "unit": "GTEPS",
               "h2d_bytes_per_step": int((g.n + 1) * 8 + g.nnz * 4),
               "d2h_bytes_per_step": int(g.n * 4), "ms_per_step": p_ms,
               "api": f"sgr_color_host_batch over {K} steps (copies overlapped with colorings)",
               "serial": serial}

    line = {"metric": METRIC, "value": value, "unit": "GTEPS", "n_gpus": 1,
            "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": ms,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "int32", "data": "synthetic",
            "config": bench_config(args, g),
            "rounds": st["rounds"], "num_colors": st["num_colors"],
            "A_scanned_per_nnz": st["edges_scanned"] / g.nnz,
            "B_worklist_per_n": st["vertices_processed"] / g.n,
            "vertices_per_s": g.n / (ms * 1e-3), "step_ms_min": min(step_ms),
            "wall_s_timed_region": wall, "gpu_launches": launches,
            "roofline": roofline, "clocks": clk, "e2e": e2e, "gen_s": gen_s}

    # secondary row (reading C4): the paper's own tie-break, v < w recolors v
    other = "paper" if args.tiebreak == "lowid" else "lowid"
    sec = None
    if not args.no_secondary:
        step(tiebreak=other)
        s_ms, s_st = [], None
        for i in range(3):
            flush.fill_(i)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            s_st = step(tiebreak=other).stats
            e1.record(stream)
            torch.cuda.synchronize()
            s_ms.append(e0.elapsed_time(e1))
        sec = {"tiebreak": other, "value": g.nnz / (statistics.mean(s_ms) * 1e-3) / 1e9,
               "unit": "GTEPS", "ms_per_step": statistics.mean(s_ms), "steps": 3,
               "rounds": s_st["rounds"], "num_colors": s_st["num_colors"],
               "A_scanned_per_nnz": s_st["edges_scanned"] / g.nnz}
        line["secondary"] = sec
    line["paper_context"] = dict(PAPER_CONTEXT)

    if not args.no_cpu_baseline:
        tb = 0 if args.tiebreak == "lowid" else 1
        o = oracle_run(g, tb, st["edges_scanned"], budget_s=30.0)
        a1_colors, a1_s = alg1_run(g)
        line["cpu_baseline"] = {"value": g.nnz / o["seconds"] / 1e9, "unit": "GTEPS",
                                "cores": o["cores"], "kind": "oracle", "sample": o["sample"],
                                "cpu_model": cpu_model(),
                                "threads_note": f"O2 on {o['cores']} OpenMP threads (one per "
                                                "host core); Algorithm 1 on 1 core below"}
        line["colors_vs_seq_greedy"] = {"ours": st["num_colors"], "alg1": a1_colors,
                                        "ratio": st["num_colors"] / a1_colors,
                                        "alg1_seconds_1core": a1_s,
                                        "speedup_vs_alg1_1core": a1_s / (ms * 1e-3)}
        if sec is not None:
            sec["colors_vs_alg1"] = sec["num_colors"] / a1_colors
            sec["speedup_vs_alg1_1core"] = a1_s / (sec["ms_per_step"] * 1e-3)
        line["paper_context"]["ours_speedup_vs_sequential_alg1_1core"] = a1_s / (ms * 1e-3)
        if o["result"] is not None:
            ok = bool(np.array_equal(o["result"].colors, colors.cpu().numpy()))
            line["parity_vs_oracle_full"] = ok
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1 or args.gpus > 1 or args.dist:
        from paper_conf_ipps_licqfsty16_b200 import benchdist
        return benchdist.run(args, check=oracle_parity)
    return run_single(args)


if __name__ == "__main__":
    main()
