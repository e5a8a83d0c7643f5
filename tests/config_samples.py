"""Deterministic single-root-edge samples of the full-size BASELINE configs 3-5.

A sample is one directed data edge e = (u, v) (its index in the CSR, i.e. its
lexicographic rank): the CUDA path runs shard (rank = e, world = 2^31 - 1) -- the
one initial edge task e, expanded by the whole persistent grid with timeout
splitting -- and the oracle enumerates the matches whose root edge is e (shard
(e, 2^31 - 1), roots [u, u + 1)).  Both use the oracle's matching order, so the
root edge maps to the same two query vertices.  Edges are picked per query among
edges whose endpoint degrees sit at given percentiles and whose labels match the
first two query vertices of that order, so that the subtrees are non-trivial but
the oracle finishes in seconds.  Holds no matching arithmetic (input selection only).
"""
from __future__ import annotations

import numpy as np

WORLD = 2**31 - 1
PERCENTILES = {3: (99.0, 99.5, 99.9), 4: (99.0, 99.5, 99.9), 5: (98.0, 99.0, 99.2)}


def pick_edges(g, offs, adj, qlabels_first_two, percentiles, seed=5):
    """[(e, u, v)] one edge per percentile: deg(u), deg(v) in [P, 1.5 P], u < v, labels match."""
    deg = np.diff(offs)
    src = np.repeat(np.arange(g.n, dtype=np.int64), deg)
    rng = np.random.default_rng(seed)
    base = src < adj
    if g.labels is not None and qlabels_first_two is not None:
        la, lb = qlabels_first_two
        base &= (g.labels[src] == la) & (g.labels[adj] == lb)
    out = []
    for p in percentiles:
        lo = np.percentile(deg, p)
        hi = max(lo * 1.5, lo + 2)
        cand = np.nonzero(base & (deg[src] >= lo) & (deg[src] <= hi) & (deg[adj] >= lo) & (deg[adj] <= hi))[0]
        if len(cand) == 0:
            continue
        e = int(cand[rng.integers(len(cand))])
        out.append((e, int(src[e]), int(adj[e])))
    return out
