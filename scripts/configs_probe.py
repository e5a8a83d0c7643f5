"""Exploration (not a bench line): time queries of a BASELINE config on one GPU, on shards.
    python scripts/configs_probe.py CFG Q1,Q2,... W RANKS [POLICY] [TAU_MS]
RANKS: comma list of shard ranks (e.g. 0 or 0,1,...,7).  W = 1 runs the full count.  Prints
per-shard kernel time and count, max/mean over the ranks given (imbalance of a W-GPU run
whose shards are these), and the full-graph time estimate W * mean."""
import json
import sys
import time

import torch

import tdfs_inputs as T
import paper_conf_icde_yuan0ha0024_b200 as M

cfg = int(sys.argv[1])
qn = sys.argv[2].split(",")
W = int(sys.argv[3])
ranks = [int(x) for x in sys.argv[4].split(",")]
policy = int(sys.argv[5]) if len(sys.argv) > 5 else 0
tau = float(sys.argv[6]) if len(sys.argv) > 6 else 10.0
flags = int(sys.argv[7]) if len(sys.argv) > 7 else 0
with_stats = len(sys.argv) > 8 and sys.argv[8] == "stats"  # instrumented kernel: tasks, warp-exit tail
t0 = time.time()
g = T.config_graph(cfg)
tg = time.time() - t0
t0 = time.time()
h = M.tdfs_load_edges(g.n, g.edges, g.labels)
torch.cuda.synchronize()
print(f"config {cfg}: gen {tg:.1f}s load {time.time() - t0:.1f}s {h.info()} W={W} policy={policy} tau={tau}", flush=True)
out = {}
for name in qn:
    q = T.labeled_query(name, 8) if cfg == 4 else T.query(name)
    p = M.plan_from_query(q)
    ts, cs = [], []
    for r in ranks:
        o = M.default_opts(shard_rank=r, shard_world=W, shard_policy=policy, chunk=8 if q.k <= 3 else 1,
                           tau_ms=None if tau < 0 else tau, flags=flags)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        c = M.tdfs_count(h, p, o)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        cs.append(c)
        extra = ""
        if with_stats:
            c2, st = M.tdfs_count(h, p, o, stats=True)
            assert c2 == c
            extra = (f"  [stats: {st['kernel_ms']:.0f} ms, enq {st['tasks_enqueued']}, timeouts {st['timeouts']}, "
                     f"warp exit first/mean/last {st['warp_exit_first_ns'] / 1e6:.0f}/{st['warp_exit_mean_ns'] / 1e6:.0f}/"
                     f"{st['warp_exit_last_ns'] / 1e6:.0f} ms, pages {st['pages_used']}]")
        print(f"  {name:14s} shard {r}/{W}: count {c:>18d}  {ts[-1]:10.1f} ms{extra}", flush=True)
    mean = sum(ts) / len(ts)
    print(f"  {name:14s} max/mean {max(ts) / mean:.3f}  est. full {W * mean / 1000:.1f} s  "
          f"shard-sum {sum(cs)}", flush=True)
    out[name] = {"ms": ts, "counts": cs, "W": W, "policy": policy}
tag = f"c{cfg}_W{W}_p{policy}_f{flags}"
json.dump(out, open(f"gpurun_out/probe_{tag}.json", "w"), indent=1)
