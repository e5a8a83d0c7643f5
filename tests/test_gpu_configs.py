"""BASELINE.json configs 3-5 at full size, in the bench launch configuration (default grid,
tau = 10 ms, 8 KB pages): the CUDA path runs sampled shards of the directed root edges
(PAPER.md:522's round-robin rule) and the oracle computes exactly the matches rooted at
the same edges (same order, so the same root edges).  Integer results: bit-exact."""
import os

import pytest

import oracle as O
import tdfs_inputs as T
from tests import gpu_util as U

pytestmark = pytest.mark.gpu
THREADS = max(1, min(64, os.cpu_count() or 1))

SAMPLES = {3: (1009, (0, 500)), 4: (1009, (0, 731)), 5: (20011, (0, 9973))}
_cache = {}


def _cfg(cfg):
    if cfg not in _cache:
        g = T.config_graph(cfg)
        _cache[cfg] = (g, O.OracleGraph(g))
    return _cache[cfg]


def _queries(cfg):
    return [(n, T.labeled_query(n, 8) if cfg == 4 else T.query(n)) for n in T.CONFIG_QUERIES[cfg]]


@pytest.mark.parametrize("cfg", [3, 4, 5])
def test_config_full_size_sampled_shards(cfg):
    g, og = _cfg(cfg)
    W, ranks = SAMPLES[cfg]
    for name, q in _queries(cfg):
        order = O.oracle_order(q)
        for r in ranks:
            got = U.count(g, q, "auto", order=order, shard_rank=r, shard_world=W)
            ref = O.count(og, q, "auto", order=order, shard=(r, W), threads=THREADS)
            assert got == ref, (cfg, name, r, got, ref)


@pytest.mark.parametrize("cfg", [3, 5])
def test_config_planner_order_equals_oracle_order_on_shard_sums(cfg):
    """The planner's own order (what bench.py runs) and the oracle's order give the same
    count over a union of shards (the shard sets differ by order, their sums do not)."""
    g, _ = _cfg(cfg)
    W = 97
    for name, q in _queries(cfg)[:2]:
        a = sum(U.count(g, q, "auto", shard_rank=r, shard_world=W) for r in range(W))
        b = sum(U.count(g, q, "auto", order=O.oracle_order(q), shard_rank=r, shard_world=W) for r in range(W))
        assert a == b, (cfg, name)
