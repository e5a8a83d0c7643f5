"""Exploration (not a bench line): time queries of a config under option variants.
    python scripts/exp_time.py CFG QUERIES VARIANTS [W]
VARIANTS: ';'-separated, each 'ENV=VAL,ENV=VAL|flags' (flags = tdfs_run_opts.flags int), '-' = defaults.
Counts of every variant must equal the first variant's (checked)."""
import json, os, sys, time
import torch
import tdfs_inputs as T
import paper_conf_icde_yuan0ha0024_b200 as M

cfg = int(sys.argv[1])
qn = sys.argv[2].split(",")
variants = sys.argv[3].split(";")
W = int(sys.argv[4]) if len(sys.argv) > 4 else 1
reps = int(os.environ.get("REPS", "2"))
g = T.config_graph(cfg)
h = M.tdfs_load_edges(g.n, g.edges, g.labels)
torch.cuda.synchronize()
res = {}
for name in qn:
    q = T.labeled_query(name, 8) if cfg == 4 else T.query(name)
    p = M.plan_from_query(q)
    ref = None
    for var in variants:
        env, _, fl = var.partition("|")
        saved = {}
        if env and env != "-":
            for kv in env.split(","):
                k, v = kv.split("=")
                saved[k] = os.environ.get(k)
                os.environ[k] = v
        kw = {}
        for kv in os.environ.get("EXP_OPTS", "").split(","):  # e.g. EXP_OPTS=chunk=32,tau_ms=1
            if kv:
                k, v = kv.split("=")
                kw[k] = float(v) if "." in v else int(v)
        o = M.default_opts(flags=int(fl or 0), shard_world=W, **kw)
        ts = []
        for r in range(reps + 1):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            c = M.tdfs_count(h, p, o)
            e1.record()
            torch.cuda.synchronize()
            if r:
                ts.append(e0.elapsed_time(e1))
        for k, v in saved.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
        ok = ref is None or c == ref
        ref = c if ref is None else ref
        res[f"{name}|{var}"] = {"count": c, "ms": min(ts), "ok": ok}
        print(f"{name:16s} {var:40s} {c:>16d} {min(ts):10.2f} ms {'OK' if ok else 'MISMATCH'}", flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open(f"gpurun_out/exp_{cfg}_{int(time.time())}.json", "w"), indent=1)
