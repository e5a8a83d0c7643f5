"""Helpers for the -m gpu tests: run the CUDA path through the C-ABI binding."""
import numpy as np

import paper_conf_icde_yuan0ha0024_b200 as M

_graph_cache = {}


def load(g):
    key = id(g)
    if key not in _graph_cache:
        _graph_cache[key] = (g, M.tdfs_load_edges(g.n, g.edges, g.labels))
    return _graph_cache[key][1]


def plan(q, order=None, constraints="auto"):
    return M.tdfs_plan_query(q.k, q.edges, q.labels, order=order, constraints=constraints)


def count(g, q, constraints="auto", order=None, stats=False, **opts):
    h = load(g)
    p = plan(q, order, constraints)
    o = M.default_opts(**opts)
    return M.tdfs_count(h, p, o, stats=stats)


def enumerate_sorted(g, q, constraints="auto", order=None, cap=None, **opts):
    h = load(g)
    p = plan(q, order, constraints)
    o = M.default_opts(**opts)
    if cap is None:
        cap = M.tdfs_count(h, p, o)
    t, total, overflow = M.tdfs_enumerate(h, p, max(cap, 1), o)
    if t.shape[0] == 0:
        return np.zeros((0, q.k), dtype=np.int32), total, overflow
    return t[np.lexsort(t.T[::-1])], total, overflow
