#!/usr/bin/env python
"""Benchmark of the T-DFS hot path on B200 (BASELINE.json metric:
"matches/sec & time-to-count per query at 1/2/4/8 B200; HBM GB/s fraction").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config 2]

Workload (N = 1): BASELINE.json configs[1] -- R-MAT scale 18, edge factor 16
(a,b,c) = (.57,.19,.19), seed 1, ids permuted -- with the queries triangle, 4-cycle,
diamond, tailed triangle and 4-clique, each counted once per step with full symmetry
breaking.  A step = the five tdfs_count jobs (one persistent kernel each).  Inputs are
resident in HBM before timing; L2 (126 MB) is flushed before every timed step because
the CSR (~32 MB) would otherwise stay cached across steps.
N > 1 (torchrun): every rank counts its round-robin shard of the directed initial edges
 and one NCCL all-reduce sums the counts -- total work is fixed: "strong".

Prints ONE JSON line (rank 0).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "matches/sec & time-to-count per query at 1/2/4/8 B200; HBM GB/s fraction"
UNIT = "matches/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--tau-ms", type=float, default=10.0)
    ap.add_argument("--chunk", type=int, default=1,
                    help="initial edge tasks per cursor grab (ABI default 8 = the paper's; 1 measured best on config 2)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--queries", type=str, default="")
    ap.add_argument("--cpu-sample-world", type=int, default=2001)
    ap.add_argument("--profile-shard-world", type=int, default=1,
                    help="profiling only: run shard 0 of W on one GPU (not a bench number)")
    ap.add_argument("--flags", type=int, default=0, help="tdfs_run_opts.flags (ablations)")
    return ap.parse_args()


def workload(cfg: int):
    import tdfs_inputs as T
    g = T.config_graph(cfg)
    names = T.CONFIG_QUERIES[cfg]
    qs = [T.labeled_query(n, 8) if cfg == 4 else T.query(n) for n in names]
    desc = {2: "R-MAT s18 EF16 (a,b,c)=(.57,.19,.19) seed 1",
            3: "R-MAT s20 EF6 seed 1", 4: "Chung-Lu n=4M gamma=2.2 dmax=15000 seed 7, 8 labels",
            5: "R-MAT s22 EF30 seed 1", 1: "ER n=2000 m=10000 seed 1"}[cfg]
    return g, qs, desc


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi sampling during the timed region (the recipe's clocks line)."""
    FIELDS = "clocks.sm,clocks.max.sm,clocks_event_reasons.active"

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            threading.Thread(target=self._read, daemon=True).start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 3:
                self.rows.append(parts)

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()
        REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
                   0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
                   0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}
        sm, mx, reasons = [], [], set()
        for a, b, c in self.rows:
            try:
                sm.append(float(a))
                mx.append(float(b))
                bits = int(c, 16)
                for k, v in REASONS.items():
                    if bits & k and v != "gpu_idle":
                        reasons.add(v)
            except ValueError:
                pass
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ helpers
def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def ncu_traffic(cfg: int):
    """dram bytes per launch of the matching kernel from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_full_summary.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    return d.get("dram_bytes_per_launch")


def cpu_baseline(g, qs, sample_world: int):
    """The oracle (as it stands) on a bounded sample: 1/sample_world of the directed root
    edges of every query, all host cores."""
    import oracle as O
    threads = os.cpu_count() or 1
    tot_m, tot_t = 0, 0.0
    for q in qs:
        t0 = time.perf_counter()
        c = O.count(g, q, "auto", shard=(0, sample_world), threads=threads)
        tot_t += time.perf_counter() - t0
        tot_m += c
    return {"value": tot_m / tot_t if tot_t > 0 else 0.0, "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": f"each query on the directed root edges with rank = 0 mod {sample_world} "
                      f"(1/{sample_world} of the initial tasks), serial Alg. 1 fanned out over roots; "
                      f"{tot_m} matches in {tot_t:.2f} s incl. adjacency build"}


# ------------------------------------------------------------------ reference arm
def run_reference(a):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    g, qs, desc = workload(a.config)
    import oracle as O
    threads = os.cpu_count() or 1
    times, matches = [], 0
    for step in range(a.warmup + a.steps):
        t0 = time.perf_counter()
        m = 0
        for q in qs:
            m += O.count(g, q, "auto", shard=(step % a.cpu_sample_world, a.cpu_sample_world), threads=threads)
        dt = time.perf_counter() - t0
        if step >= a.warmup:
            times.append(dt)
            matches += m
    tot = sum(times)
    val = matches / tot if tot else 0.0
    sample = (f"each step: every query on 1/{a.cpu_sample_world} of the directed root edges "
              f"(shard r = step mod {a.cpu_sample_world}), oracle O2 with {threads} threads")
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": 1000 * tot / max(1, a.steps), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": f"config{a.config}: {desc}", "queries": [q.name for q in qs],
                       "constraints": "full symmetry breaking", "sampled": True},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def run_ours(a):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_icde_yuan0ha0024_b200 as M
    from paper_conf_icde_yuan0ha0024_b200 import dist as D

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        D.init_process_group("nccl")
    torch.cuda.set_device(local)
    dev = local
    stream = torch.cuda.current_stream(dev)

    g, qs, desc = workload(a.config)
    if a.queries:
        keep = set(a.queries.split(","))
        qs = [q for q in qs if q.name in keep or q.name.replace("_lab", "") in keep]
    t_load0 = time.perf_counter()
    h = M.tdfs_load_edges(g.n, g.edges, g.labels, device=dev)
    torch.cuda.synchronize()
    load_s = time.perf_counter() - t_load0
    info = h.info()
    t_plan0 = time.perf_counter()
    plans = [M.plan_from_query(q) for q in qs]
    plan_s = time.perf_counter() - t_plan0
    tau = None if a.tau_ms < 0 else a.tau_ms
    # per query: k = 3 jobs are one intersection per edge task, so they keep the paper's chunk of 8
    # (one cursor atomic per edge costs the triangle 4.8 -> 17.4 ms); deeper queries take a.chunk
    qopts = [M.default_opts(tau_ms=tau, chunk=(8 if q.k <= 3 else a.chunk), shard_rank=rank,
                            shard_world=world * a.profile_shard_world, flags=a.flags) for q in qs]
    ws_bytes = max(M.tdfs_workspace_bytes(h, p, o) for p, o in zip(plans, qopts))
    ws = torch.empty(ws_bytes, dtype=torch.uint8, device=f"cuda:{dev}")
    d_counts = torch.zeros(len(qs), dtype=torch.int64, device=f"cuda:{dev}")
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=f"cuda:{dev}")

    # W (algorithmic adjacency bytes) per query from one instrumented run (untimed)
    W, Wfull, stats_runs = [], [], []
    for p in plans:
        c, st = M.tdfs_count(h, p, qopts[len(W)], workspace=ws, stats=True)
        W.append(st["stream_bytes"])   # roofline bytes, R29b
        Wfull.append(st["adj_bytes"])  # SURVEY 8(d) full-operand W, for reference
        stats_runs.append(st)

    def step(ev_q=None):
        for i, p in enumerate(plans):
            if ev_q is not None:
                ev_q[i][0].record(stream)
            M.tdfs_count(h, p, qopts[i], workspace=ws, stream=stream, d_count=d_counts[i:i + 1], sync=False)
            if ev_q is not None:
                ev_q[i][1].record(stream)
        if world > 1:
            dist.all_reduce(d_counts)

    for _ in range(a.warmup):
        flush.zero_()
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    clocks = ClockSampler(dev)
    clocks.start()
    step_ms, q_ms = [], [[] for _ in qs]
    counts = None
    for s in range(a.steps):
        flush.zero_()  # L2 flush, outside the timed interval
        ev0 = torch.cuda.Event(enable_timing=True)
        ev1 = torch.cuda.Event(enable_timing=True)
        evq = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in qs]
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ev0.record(stream)
        step(evq)
        ev1.record(stream)
        torch.cuda.synchronize()
        step_ms.append(ev0.elapsed_time(ev1))
        for i, (e0, e1) in enumerate(evq):
            q_ms[i].append(e0.elapsed_time(e1))
        counts = d_counts.cpu().tolist()
    clk = clocks.stop()
    M.tdfs_workspace_status(ws, stream, dev)

    total_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=f"cuda:{dev}")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
        qt = torch.tensor([sum(x) for x in q_ms], dtype=torch.float64, device=f"cuda:{dev}")
        dist.all_reduce(qt, op=dist.ReduceOp.MAX)
        q_tot = qt.tolist()
    else:
        q_tot = [sum(x) for x in q_ms]
    matches_per_step = int(sum(counts))
    value = matches_per_step * a.steps / (total_ms / 1000.0)

    # roofline of the dominant kernel (the matching kernel; 1 launch per query per step)
    peak, peak_kind = measured_peaks()
    w_local = sum(W)  # this rank's shard bytes per step
    per_launch_bytes = w_local / len(qs)
    avg_launch_s = (sum(q_tot) / len(qs)) / a.steps / 1000.0
    achieved = per_launch_bytes / avg_launch_s / 1e9
    traffic = ncu_traffic(a.config)

    # e2e through the public API with host buffers: H2D of the CSR from pinned memory,
    # load, plan, the five counts, D2H of the counts -- every step
    e2e = None
    if not a.no_e2e:
        import tdfs_inputs as T
        offs_np, adj_np = T.to_csr(g)
        offs_h = torch.from_numpy(offs_np).pin_memory()
        adj_h = torch.from_numpy(adj_np).pin_memory()
        lab_h = None if g.labels is None else torch.from_numpy(g.labels).pin_memory()
        h2d = offs_h.numel() * 8 + adj_h.numel() * 4 + (0 if lab_h is None else lab_h.numel())
        e2e_t = []
        for s in range(a.warmup + a.steps):
            flush.zero_()
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            t0 = time.perf_counter()
            hh = M.tdfs_load_graph(offs_h.numpy(), adj_h.numpy(), None if lab_h is None else lab_h.numpy(),
                                   device=dev)
            pl = [M.plan_from_query(q) for q in qs]
            tot = 0
            dc = torch.zeros(len(qs), dtype=torch.int64, device=f"cuda:{dev}")
            for i, p in enumerate(pl):
                M.tdfs_count(hh, p, qopts[i], workspace=ws, stream=stream, d_count=dc[i:i + 1], sync=False)
            if world > 1:
                dist.all_reduce(dc)
            tot = int(dc.cpu().sum().item())
            dt = time.perf_counter() - t0
            hh.free()
            if s >= a.warmup:
                e2e_t.append(dt)
        et = sum(e2e_t)
        if world > 1:
            t = torch.tensor([et], dtype=torch.float64, device=f"cuda:{dev}")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            et = float(t.item())
        e2e = {"value": matches_per_step * a.steps / et, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": 8 * len(qs),
               "includes": "tdfs_load_graph (H2D of pinned CSR, src build), tdfs_plan_query x5, tdfs_count x5, "
                           "D2H of the counts"}

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_baseline(g, qs, a.cpu_sample_world)

    if rank == 0:
        per_query = {}
        for i, q in enumerate(qs):
            per_query[q.name] = {"count": int(counts[i]), "time_to_count_ms": q_tot[i] / a.steps,
                                 "matches_per_s": counts[i] / (q_tot[i] / a.steps / 1000.0),
                                 "W_bytes": int(W[i]), "W_full_bytes": int(Wfull[i]),
                                 "eff_GBps": W[i] / (q_tot[i] / a.steps / 1000.0) / 1e9,
                                 "timeouts": int(stats_runs[i]["timeouts"]),
                                 "tasks_enqueued": int(stats_runs[i]["tasks_enqueued"]),
                                 "pages_used": int(stats_runs[i]["pages_used"])}
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": total_ms / a.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": f"config{a.config}: {desc}", "n": g.n, "m": info["m"], "dmax": info["dmax"],
                       "queries": [q.name for q in qs], "constraints": "full symmetry breaking (stabilizer chain)",
                       "tau_ms": a.tau_ms, "chunk": {"k3": 8, "k>=4": a.chunk}, "parallelism": f"shard{world}",
                       "l2": "flushed (256 MB write) before every timed step", "load_s": load_s, "plan_s": plan_s,
                       "per_query": per_query},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "peak_kind": peak_kind,
                         "note": "achieved = algorithmic bytes per matching-kernel launch (DESIGN.md R29b: 16 B per "
                                 "Eq.(1) operand + 4 B x smallest constraint-windowed operand, per extension; from one "
                                 "STATS run) / mean tdfs_count duration (CUDA events on the launch stream); traffic = "
                                 "ncu dram bytes per launch (profiles/ncu_full_summary.json)"},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": 4 * len(qs) * a.steps,
            "clocks": clk,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    a = parse()
    if a.impl == "reference":
        return run_reference(a)
    return run_ours(a)


if __name__ == "__main__":
    sys.exit(main())
