"""Time every BASELINE config's queries on one GPU (full graph) -- exploration, not a bench line."""
import json, sys, time
import torch
import tdfs_inputs as T
import paper_conf_icde_yuan0ha0024_b200 as M

cfgs = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else [3, 4, 5]
W = int(sys.argv[2]) if len(sys.argv) > 2 else 1
out = {}
for cfg in cfgs:
    t0 = time.time()
    g = T.config_graph(cfg)
    tg = time.time() - t0
    t0 = time.time()
    h = M.tdfs_load_edges(g.n, g.edges, g.labels)
    torch.cuda.synchronize()
    tl = time.time() - t0
    info = h.info()
    print(f"config {cfg}: gen {tg:.1f}s load {tl:.1f}s {info}", flush=True)
    for name in T.CONFIG_QUERIES[cfg]:
        q = T.labeled_query(name, 8) if cfg == 4 else T.query(name)
        p = M.plan_from_query(q)
        o = M.default_opts(shard_world=W)
        t0 = time.time()
        try:
            c, st = M.tdfs_count(h, p, o, stats=True)
            dt = time.time() - t0
            print(f"  {name:12s} count {c:>16d}  {dt*1000:9.1f} ms  kernel {st['kernel_ms']:9.1f} ms  "
                  f"enq {st['tasks_enqueued']} pages {st['pages_used']}/{st['pool_pages']}", flush=True)
            out[f"{cfg}/{name}"] = {"count": c, "ms": st["kernel_ms"], "shard_world": W}
        except M.TdfsError as e:
            print(f"  {name}: {e}", flush=True)
    del h
json.dump(out, open(f"gpurun_out/configs_probe_{'_'.join(map(str, cfgs))}_W{W}.json", "w"), indent=1)
