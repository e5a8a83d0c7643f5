"""Exploration (not a bench line): time queries of a config with whichever libtdfs.so the
package on sys.path carries (PYTHONPATH=/tmp/var_X:$PWD, see variants.sh).  Median of REPS.
    python scripts/variant_time.py CFG Q1,Q2 [REPS] [W] [HUB_MB] [deg]"""
import os
import statistics
import sys

import torch

import tdfs_inputs as T
import paper_conf_icde_yuan0ha0024_b200 as M

cfg = int(sys.argv[1])
qn = sys.argv[2].split(",")
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
W = int(sys.argv[4]) if len(sys.argv) > 4 else 1
hub_mb = int(sys.argv[5]) if len(sys.argv) > 5 else 0
degree_order = len(sys.argv) > 6 and sys.argv[6] == "deg"
g = T.config_graph(cfg)
h = M.tdfs_load_edges(g.n, g.edges, g.labels, hub_bitmap_bytes=hub_mb << 20 if hub_mb > 0 else hub_mb,
                      degree_order=degree_order)
torch.cuda.synchronize()
print(f"lib {M.LIB_PATH} hub_mb {hub_mb} degree_order {degree_order}", flush=True)
for name in qn:
    q = T.labeled_query(name, 8) if cfg == 4 else T.query(name)
    p = M.plan_from_query(q)
    o = M.default_opts(chunk=8 if q.k <= 3 else int(os.environ.get("CHUNK", "1")), shard_world=W,
                       tau_ms=float(os.environ.get("TAU", "10")))
    ts = []
    for r in range(reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        c = M.tdfs_count(h, p, o)
        e1.record()
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    print(f"  {name:16s} {statistics.median(ts):10.2f} ms  count {c}", flush=True)
