"""Small adversarial runs of the CUDA path for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): tau = 0 (split at every eligible step), a 1-task queue (queue_ints = 3: every push
races for one slot), 128-byte pages (a level crosses a page every 32 ids), 2 ranks' shards, the
degree-balanced partition, leaf staging on and off, the streaming enumerate ring, range tasks at
levels 2-4.  Counts are checked against the oracle (test infrastructure).
    compute-sanitizer --tool memcheck python scripts/sanitize_cases.py"""
import sys

import numpy as np

import oracle as O
import tdfs_inputs as T
import paper_conf_icde_yuan0ha0024_b200 as M

g = T.rmat(7, 6, 3)
h = M.tdfs_load_edges(g.n, g.edges)
cases = 0
for name in ["triangle", "c4", "diamond", "tailed_triangle", "k4", "house", "c5", "w6"]:
    q = T.query(name)
    ref = O.count(g, q, "auto")
    p = M.plan_from_query(q)
    for kw in (dict(tau_ms=0.0, queue_ints=3, page_bytes=128, blocks=2, warps_per_block=4),
               dict(tau_ms=0.0, page_bytes=128, flags=M.TDFS_RUN_NO_LEAF_STAGE),
               dict(tau_ms=0.0, queue_ints=30, flags=M.TDFS_RUN_NO_RANGE_TASKS),
               dict(tau_ms=0.001, chunk=3)):
        got = M.tdfs_count(h, p, M.default_opts(**kw))
        assert got == ref, (name, kw, got, ref)
        cases += 1
    got = sum(M.tdfs_count(h, p, M.default_opts(tau_ms=0.0, shard_rank=r, shard_world=2,
                                                shard_policy=M.TDFS_SHARD_DEGREE_BALANCED)) for r in range(2))
    assert got == ref, (name, "shards", got, ref)
    parts = []
    tot = M.tdfs_enumerate_stream(h, p, lambda a: parts.append(a), 64, M.default_opts(tau_ms=0.0, queue_ints=30))
    t = np.concatenate(parts) if parts else np.zeros((0, q.k), np.int32)
    assert tot == ref == t.shape[0], (name, "stream", tot, ref)
    cases += 2
print(f"sanitize cases ok: {cases}")
sys.exit(0)
