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
N > 1 (torchrun): every rank counts its shard of the directed initial edges (round-robin,
PAPER.md:522, or --shard-policy 1 degree-balanced, R31; or --shared-cursor: all ranks
take edge chunks from one cursor in rank 0's HBM, NEXT-3) and one NCCL all-reduce of
{count, failed} sums the counts -- total work is fixed: "strong".

--config 3/4/5: the gated query sets of tdfs_inputs.BENCH_QUERIES with the per-config timeout tau
(TAU_DEFAULT_MS) and hub-bitmap budget (HUB_MB_DEFAULT) that this repo's sweeps found best (R37, section 10).
The roofline object reports the dominant launch: R32 algorithmic bytes / its CUDA-event time against the measured
HBM peak, the same-source ncu DRAM traffic, and (config 2) its L2 sector rate against the measured L2 peaks.

After timing, the counts are checked against the oracle goldens of the config
(tests/golden/c<cfg>_counts.txt, written by scripts/golden_counts.py from oracle/ only) when
the file has them; a mismatch or a failed job (TDFS_COUNT_INVALID) aborts the run.

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


# timeout tau per config (PAPER.md:486-518 tunes tau per dataset; 10 ms is the paper's choice): measured on
# one B200 -- C4 prism/w5 1 ms (33.0 / 12.7 s vs 36.6 / 14.0 s at 10 ms), C5 k4 100 ms (1/16 shard 2.66 s vs
# 3.85 s at 10 ms, 5.31 s at 1 ms); profiles/c4_splitting_diag_r02.txt, profiles/c45_r02o.log
# C3 k5 100 ms (723 vs 868 ms at 10 ms, profiles/tau_r02aa.log); C2's five-query step is flat over 10-100 ms
TAU_DEFAULT_MS = {3: 100.0, 4: 1.0, 5: 100.0}
# hub-bitmap budget per config (MB; library default 256 MB): measured on one B200 (profiles/hub_budget_r02s.log,
# 256 MB / 1 / 4 / 16 GB): C5 k4 1/16 shard 2.66 / 2.14 / 2.20 / 2.46 s, C4 prism 1/64 0.79 / 0.69 / 0.76 / 0.74 s,
# w5 flat; C3 c5 16.5 / 18.8 s (more bitmaps than the lists they replace thrash L2), C3 k5 flat
HUB_MB_DEFAULT = {4: 1024, 5: 1024}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--tau-ms", type=float, default=None,
                    help="timeout tau (ms, < 0 = none); default per config: TAU_DEFAULT_MS (measured sweeps, DESIGN.md 10)")
    ap.add_argument("--chunk", type=int, default=1,
                    help="initial edge tasks per cursor grab (ABI default 8 = the paper's; 1 measured best on config 2)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--queries", type=str, default="")
    ap.add_argument("--cpu-sample-world", type=int, default=2001)
    ap.add_argument("--profile-shard-world", type=int, default=1,
                    help="profiling only: run shard 0 of W on one GPU (not a bench number)")
    ap.add_argument("--flags", type=int, default=0, help="tdfs_run_opts.flags (ablations)")
    ap.add_argument("--shard-policy", type=int, default=0, help="N > 1: 0 round-robin (paper), 1 degree-balanced")
    ap.add_argument("--shared-cursor", action="store_true", help="N > 1: cross-GPU shared chunk cursor (NEXT-3)")
    ap.add_argument("--hub-bitmap-mb", type=int, default=None,
                    help="hub bitmap budget (0 = library default); default per config: HUB_MB_DEFAULT")
    ap.add_argument("--degree-order", action="store_true",
                    help="load with TDFS_GRAPH_DEGREE_ORDER (symmetry breaking by degree rank, DESIGN.md R35)")
    ap.add_argument("--also-degree-order", type=int, default=1,
                    help="1: also time the queries on the degree-ordered graph (reported under degree_order)")
    ap.add_argument("--no-stats", action="store_true",
                    help="skip the instrumented run (no roofline bytes): long configs-3..5 queries")
    return ap.parse_args()


def workload(cfg: int):
    import tdfs_inputs as T
    g = T.config_graph(cfg)
    names = T.BENCH_QUERIES[cfg]
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


def kernel_source_hash() -> str:
    """sha256 of the product's CUDA/C++ sources: ties a committed ncu summary to the kernel build."""
    import hashlib
    h = hashlib.sha256()
    csrc = os.path.join(ROOT, "paper_conf_icde_yuan0ha0024_b200", "csrc")
    for f in sorted(os.listdir(csrc)) + ["../../include/tdfs.h"]:
        with open(os.path.join(csrc, f), "rb") as fh:
            h.update(fh.read())
    return h.hexdigest()[:16]


def ncu_summary(cfg: int):
    """Per-query ncu --set full numbers of THIS kernel build (profiles/ncu_full_summary.json,
    written by scripts/ncu_summary.py with the source hash); None when the build differs."""
    p = os.path.join(ROOT, "profiles", "ncu_full_summary.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    if d.get("source_hash") != kernel_source_hash() or d.get("config") != cfg:
        return None
    return d


def goldens(cfg: int):
    p = os.path.join(ROOT, "tests", "golden", f"c{cfg}_counts.txt")
    out = {}
    if os.path.exists(p):
        for line in open(p):
            if line.strip() and not line.startswith("#"):
                k, v = line.split(":", 1)
                out[k.strip()] = int(v.split()[0])
    return out


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_baseline(g, qs, sample_world: int):
    """The oracle (as it stands) on a bounded sample: 1/sample_world of the directed root
    edges of every query, all host cores; plus the single-threaded oracle on 1/(10 W)."""
    import oracle as O
    threads = os.cpu_count() or 1
    og = O.OracleGraph(g)
    tot_m, tot_t = 0, 0.0
    for q in qs:
        t0 = time.perf_counter()
        c = O.count(og, q, "auto", shard=(0, sample_world), threads=threads)
        tot_t += time.perf_counter() - t0
        tot_m += c
    w1 = 10 * sample_world + 1
    one_m, one_t = 0, 0.0
    for q in qs:
        t0 = time.perf_counter()
        one_m += O.count(og, q, "auto", shard=(0, w1), threads=1)
        one_t += time.perf_counter() - t0
    return {"value": tot_m / tot_t if tot_t > 0 else 0.0, "unit": UNIT, "cores": threads, "kind": "oracle",
            "cpu_model": cpu_model(),
            "single_core_value": one_m / one_t if one_t > 0 else 0.0,
            "sample": f"each query on the directed root edges with rank = 0 mod {sample_world} "
                      f"(1/{sample_world} of the initial tasks), serial Alg. 1 fanned out over roots; "
                      f"{tot_m} matches in {tot_t:.2f} s; single core: 1/{w1} of the root edges, "
                      f"{one_m} matches in {one_t:.2f} s"}


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
    if a.hub_bitmap_mb is None:
        a.hub_bitmap_mb = HUB_MB_DEFAULT.get(a.config, 0)
    hub_bytes = a.hub_bitmap_mb << 20
    t_load0 = time.perf_counter()
    h = M.tdfs_load_edges(g.n, g.edges, g.labels, device=dev, hub_bitmap_bytes=hub_bytes, degree_order=a.degree_order)
    torch.cuda.synchronize()
    load_s = time.perf_counter() - t_load0
    info = h.info()
    t_plan0 = time.perf_counter()
    plans = [M.plan_from_query(q) for q in qs]
    plan_s = time.perf_counter() - t_plan0
    if a.tau_ms is None:
        a.tau_ms = TAU_DEFAULT_MS.get(a.config, 10.0)
    tau = None if a.tau_ms < 0 else a.tau_ms
    cursors = D.SharedCursorGroup(dev) if (world > 1 and a.shared_cursor) else None
    # per query: k = 3 jobs are one intersection per edge task, so they keep the paper's chunk of 8
    # (one cursor atomic per edge costs the triangle 4.8 -> 17.4 ms); deeper queries take a.chunk
    qopts = [M.default_opts(tau_ms=tau, chunk=(8 if q.k <= 3 else a.chunk), shard_rank=rank,
                            shard_world=world * a.profile_shard_world, shard_policy=a.shard_policy,
                            flags=a.flags) for q in qs]
    if cursors is not None:
        for o in qopts:
            o.shared_cursor = cursors.cursor.ptr
    ws_bytes = max(M.tdfs_workspace_bytes(h, p, o) for p, o in zip(plans, qopts))
    ws = torch.empty(ws_bytes, dtype=torch.uint8, device=f"cuda:{dev}")
    d_counts = torch.zeros(len(qs), dtype=torch.int64, device=f"cuda:{dev}")
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=f"cuda:{dev}")

    # roofline bytes (R32) and W per query from one instrumented run (untimed;
    # with a shared cursor the STATS run takes this rank's static shard instead)
    W, Wfull, stats_runs = [], [], []
    for p, o in zip(plans, qopts):
        if a.no_stats:
            W.append(0)
            Wfull.append(0)
            stats_runs.append({"timeouts": -1, "tasks_enqueued": -1, "pages_used": -1, "nodes_per_level": [],
                               "warp_exit_first_ns": 0, "warp_exit_mean_ns": 0, "warp_exit_last_ns": 0})
            continue
        so = M.tdfs_run_opts.from_buffer_copy(o)
        so.shared_cursor = None
        c, st = M.tdfs_count(h, p, so, workspace=ws, stats=True)
        W.append(st["stream_bytes"])
        Wfull.append(st["adj_bytes"])
        stats_runs.append(st)

    def launch(i, ev_q=None):
        if ev_q is not None:
            ev_q[i][0].record(stream)
        M.tdfs_count(h, plans[i], qopts[i], workspace=ws, stream=stream, d_count=d_counts[i:i + 1], sync=False)
        if ev_q is not None:
            ev_q[i][1].record(stream)

    def step(ev_q=None):
        for i in range(len(plans)):
            if cursors is not None:
                cursors.prepare(stream)  # zero the shared cursor, fence all ranks (host sync)
            launch(i, ev_q)
            if cursors is not None:
                cursors.finish()

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
        if world > 1:  # the one exchange: {count, failed} per query (checked)
            summed = D.reduce_counts(d_counts.clone())
        ev1.record(stream)
        torch.cuda.synchronize()
        step_ms.append(ev0.elapsed_time(ev1))
        for i, (e0, e1) in enumerate(evq):
            q_ms[i].append(e0.elapsed_time(e1))
        local_counts = d_counts.cpu().tolist()
        if any(c == D.COUNT_INVALID_I64 for c in local_counts):  # a failed job is an error, never a count
            raise RuntimeError(f"tdfs job failed (TDFS_COUNT_INVALID) in step {s}: {local_counts}")
        counts = summed.cpu().tolist() if world > 1 else local_counts
    clk = clocks.stop()
    M.tdfs_workspace_status(ws, stream, dev)

    total_ms = sum(step_ms)
    q_med = [statistics.median(x) for x in q_ms]
    if world > 1:
        t = torch.tensor([total_ms] + [sum(x) for x in q_ms] + q_med, dtype=torch.float64, device=f"cuda:{dev}")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        tl = t.tolist()
        total_ms, q_tot, q_med = tl[0], tl[1:1 + len(qs)], tl[1 + len(qs):]
    else:
        q_tot = [sum(x) for x in q_ms]
    matches_per_step = int(sum(counts))
    value = matches_per_step * a.steps / (total_ms / 1000.0)

    # parity: every full count equals the oracle golden of this config (when present)
    gold = goldens(a.config) if a.profile_shard_world == 1 else {}  # counts are full counts (all-reduced)
    parity = {}
    for i, q in enumerate(qs):
        gname = q.name.replace("_lab", "")
        if gname in gold:
            if counts[i] != gold[gname]:
                raise RuntimeError(f"count mismatch vs oracle golden for {gname}: {counts[i]} != {gold[gname]}")
            parity[gname] = "equal to oracle golden"

    # roofline of the dominant kernel: the matching launch of the slowest query (one launch per
    # query per step); achieved = its R32 bytes per launch / its mean launch time (CUDA events)
    peak, peak_kind = measured_peaks()
    dom = max(range(len(qs)), key=lambda i: q_tot[i])
    dom_s = q_tot[dom] / a.steps / 1000.0
    achieved = W[dom] / dom_s / 1e9
    ncu = ncu_summary(a.config)
    traffic, l2 = None, None
    if ncu is not None and qs[dom].name in ncu.get("per_query", {}):
        nq = ncu["per_query"][qs[dom].name]
        traffic = nq.get("dram_bytes")
        if nq.get("lts_bytes") is not None:
            dur = nq["duration_ms"] / 1000.0
            l2 = {"lts_t_bytes": nq["lts_bytes"], "ncu_duration_ms": nq.get("duration_ms"),
                  "achieved_GBps": nq["lts_bytes"] / dur / 1e9,
                  "peak_GBps": ncu.get("l2_peak_gbs"), "l2_hit_rate": nq.get("l2_hit"),
                  "frac": (nq["lts_bytes"] / dur / 1e9) / ncu["l2_peak_gbs"] if ncu.get("l2_peak_gbs") else None}
            if nq.get("lts_read_sectors_sm") is not None and ncu.get("l2_random_sectors_per_ns"):
                # the kernel's reads are scattered probes: compare the L2->SM sector rate with the measured
                # rate of random 32-B sector reads from an L2-resident buffer (scripts/l2_peak.cu)
                rate = nq["lts_read_sectors_sm"] / dur / 1e9
                l2.update({"read_sectors_per_ns": rate, "peak_random_sectors_per_ns": ncu["l2_random_sectors_per_ns"],
                           "frac_random_sectors": rate / ncu["l2_random_sectors_per_ns"]})

    # e2e through the public API with host buffers: H2D of the CSR from pinned memory,
    # load, plan, the counts, D2H of the counts -- every step
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
                                   device=dev, hub_bitmap_bytes=hub_bytes, degree_order=a.degree_order)
            pl = [M.plan_from_query(q) for q in qs]
            dc = torch.zeros(len(qs), dtype=torch.int64, device=f"cuda:{dev}")
            for i, p in enumerate(pl):
                if cursors is not None:
                    cursors.prepare(stream)
                M.tdfs_count(hh, p, qopts[i], workspace=ws, stream=stream, d_count=dc[i:i + 1], sync=False)
                if cursors is not None:
                    cursors.finish()
            tot = D.reduce_counts(dc)  # checked (and all-reduced for N > 1)
            tot = int(tot.sum().item())
            dt = time.perf_counter() - t0
            hh.free()
            if s >= a.warmup:
                e2e_t.append(dt)
            assert tot == matches_per_step, (tot, matches_per_step)
        et = sum(e2e_t)
        if world > 1:
            t = torch.tensor([et], dtype=torch.float64, device=f"cuda:{dev}")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            et = float(t.item())
        e2e = {"value": matches_per_step * a.steps / et, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": 8 * len(qs),
               "includes": f"tdfs_load_graph (H2D of pinned CSR, src array, hub bitmaps), tdfs_plan_query x{len(qs)}, "
                           f"tdfs_count x{len(qs)}, checked reduce + D2H of the counts"}

    # the same queries on the degree-ordered graph (TDFS_GRAPH_DEGREE_ORDER, R35): same counts,
    # symmetry broken by degree rank -- reported next to the headline (which stays the paper's id order)
    deg = None
    # (a profiling shard of the renumbered graph holds other root edges: compare only whole-graph counts)
    if a.also_degree_order and not a.degree_order and cursors is None and a.profile_shard_world == 1:
        hd = M.tdfs_load_edges(g.n, g.edges, g.labels, device=dev, hub_bitmap_bytes=hub_bytes, degree_order=True)
        dws_bytes = max(M.tdfs_workspace_bytes(hd, p, o) for p, o in zip(plans, qopts))
        dws = ws if dws_bytes <= ws.numel() else torch.empty(dws_bytes, dtype=torch.uint8, device=f"cuda:{dev}")
        dc = torch.zeros(len(qs), dtype=torch.int64, device=f"cuda:{dev}")
        dq = [[] for _ in qs]
        for s in range(a.warmup + a.steps):
            flush.zero_()
            torch.cuda.synchronize()
            for i, p in enumerate(plans):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                M.tdfs_count(hd, p, qopts[i], workspace=dws, stream=stream, d_count=dc[i:i + 1], sync=False)
                e1.record(stream)
                torch.cuda.synchronize()
                if s >= a.warmup:
                    dq[i].append(e0.elapsed_time(e1))
            dcounts = D.reduce_counts(dc.clone()).cpu().tolist()
            if dcounts != counts:
                raise RuntimeError(f"degree-ordered counts differ: {dcounts} vs {counts}")
        dtot = sum(sum(x) for x in dq) / a.steps
        deg = {"ms_per_step": dtot, "value": matches_per_step / (dtot / 1000.0), "unit": UNIT,
               "counts": "equal to the id-order counts (checked every step)",
               "per_query_ms": {q.name: sum(dq[i]) / a.steps for i, q in enumerate(qs)}}
        hd.free()

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_baseline(g, qs, a.cpu_sample_world)

    if rank == 0:
        per_query = {}
        for i, q in enumerate(qs):
            t_s = q_tot[i] / a.steps / 1000.0
            per_query[q.name] = {"count": int(counts[i]), "time_to_count_ms": q_tot[i] / a.steps,
                                 "time_to_count_median_ms": q_med[i],
                                 "matches_per_s": counts[i] / t_s,
                                 "roofline_bytes": int(W[i]), "W_full_bytes": int(Wfull[i]),
                                 "eff_GBps": W[i] / t_s / 1e9, "frac": W[i] / t_s / 1e9 / peak,
                                 "timeouts": int(stats_runs[i]["timeouts"]),
                                 "tasks_enqueued": int(stats_runs[i]["tasks_enqueued"]),
                                 "pages_used": int(stats_runs[i]["pages_used"]),
                                 "warp_exit_ms_first_mean_last_stats_run": [
                                     round(stats_runs[i][f"warp_exit_{x}_ns"] / 1e6, 3) for x in ("first", "mean", "last")],
                                 "nodes_per_level": stats_runs[i]["nodes_per_level"][:q.k]}
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": total_ms / a.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": f"config{a.config}: {desc}", "n": g.n, "m": info["m"], "dmax": info["dmax"],
                       "queries": [q.name for q in qs],
                       "constraints": "full symmetry breaking (stabilizer chain)" +
                                      (" on degree ranks (TDFS_GRAPH_DEGREE_ORDER)" if a.degree_order else " on vertex ids"),
                       "tau_ms": a.tau_ms, "hub_bitmap_mb": a.hub_bitmap_mb or 256, "chunk": {"k3": 8, "k>=4": a.chunk},
                       "parallelism": f"shard{world}" + ("-shared-cursor" if cursors is not None else
                                                         f"-policy{a.shard_policy}"),
                       "l2": "flushed (256 MB write) before every timed step", "load_s": load_s, "plan_s": plan_s,
                       "parity": parity or "no goldens for this config / shard", "per_query": per_query},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "peak_kind": peak_kind,
                         "kernel": f"tdfs_kernel<0,0> ({qs[dom].name}, the dominant launch)",
                         "l2": l2,
                         "note": "achieved = algorithmic bytes of the dominant matching launch (DESIGN.md R32: per "
                                 "extension 16 B per Eq.(1) operand + 4 B x the smallest constraint-windowed Eq.(1) "
                                 "source, 0 for a count-only last position; one STATS run) / its mean tdfs_count "
                                 "duration (CUDA events on the launch stream); traffic = ncu dram bytes of that "
                                 "launch from profiles/ncu_full_summary.json of this source hash (else null)"},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": 4 * len(qs) * a.steps,
            "clocks": clk,
            "degree_order": deg,
        }
        print(json.dumps(line), flush=True)
    if cursors is not None:
        cursors.close()
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
