"""The paper's mechanisms exercised one by one on the device (through tdfs_test.h):
Q_task (Alg. 3), the paged stack writer (Alg. 5, Fig. 6) and the timeout split (Fig. 5)."""
import numpy as np
import pytest

import oracle as O
import tdfs_inputs as T
import paper_conf_icde_yuan0ha0024_b200 as M
from tests import gpu_util as U

pytestmark = pytest.mark.gpu


def _tasks(n, seed=0):
    rng = np.random.default_rng(seed)
    t = rng.integers(0, 1 << 30, size=(n, 3)).astype(np.int32)
    t[rng.random(n) < 0.3, 2] = -2  # 2-vertex tasks <v1, v2, -2>
    return t


def _sorted_rows(a):
    return a[np.lexsort(a.T[::-1])]


# ------------------------------------------------------------------ Alg. 3
@pytest.mark.parametrize("base", [0, (1 << 32) - 5, (1 << 63) - 7])
def test_queue_single_warp_fifo_full_and_empty(base):
    cap = 10
    t = _tasks(25)
    out, n_enq = M.tdfs_test_queue(0, t, cap, 1, base)
    assert n_enq == cap                      # enqueue returns false once full
    assert np.array_equal(out, t[:cap])      # FIFO; dequeue returns false once empty


@pytest.mark.parametrize("base", [0, (1 << 32) - 3, (1 << 63) - 100])
@pytest.mark.parametrize("cap,warps", [(7, 64), (1000, 512), (3, 8)])
def test_queue_multi_warp_exactly_once(base, cap, warps):
    t = _tasks(20000, seed=cap)
    out, n_enq = M.tdfs_test_queue(1, t, cap, warps, base)
    assert n_enq == t.shape[0]
    assert out.shape == t.shape
    assert np.array_equal(_sorted_rows(out), _sorted_rows(t))   # multiset in == multiset out


# ------------------------------------------------------------------ Alg. 5 / Fig. 6
def test_paged_write_fig6_example():
    """8 KB pages (2048 ids); a 32-wide batch at positions 2032-2063:
    threads 1-16 write offsets 2032-2047 of page 0, threads 17-32 offsets 0-15 of a new
    page requested for thread 17 (lane 16)."""
    r = M.tdfs_test_paged_write(8192, 2032)
    assert r["readback_ok"] == 1
    assert r["page"][:16] == [0] * 16 and r["offset"][:16] == list(range(2032, 2048))
    assert r["page"][16:] == [1] * 16 and r["offset"][16:] == list(range(0, 16))
    assert r["new_pages"] == 1
    assert r["first_lane_on_new_page"] == 16


def test_paged_write_ballot_compaction_and_min_page():
    mask = 0b1010_1010_1010_1010_1010_1010_1010_1011   # 17 valid lanes
    r = M.tdfs_test_paged_write(128, 20, mask)     # 32 ids per page; crosses at 32
    valid = [l for l in range(32) if mask >> l & 1]
    pos = [20 + i for i in range(len(valid))]
    assert [r["page"][l] for l in valid] == [p // 32 for p in pos]
    assert [r["offset"][l] for l in valid] == [p % 32 for p in pos]
    assert all(r["page"][l] == -1 for l in range(32) if not mask >> l & 1)
    assert r["new_pages"] == 1 and r["readback_ok"] == 1
    r = M.tdfs_test_paged_write(128, 0, 0xFFFFFFFF)  # a full batch fills exactly one page
    assert r["new_pages"] == 1 and r["page"] == [0] * 32


# ------------------------------------------------------------------ Fig. 5 / Alg. 4
def test_timeout_split_single_warp_trace():
    """tau = 0, one warp: every split-eligible step times out.  The trace must show
    (a) the first chunk's edges pushed as <v1, v2, -2> in chunk order, (b) tasks never
    carry more than 3 matched vertices, (c) every <v1,v2,v3> task
    is an admissible 3-prefix, and the count is unchanged."""
    g = T.rmat(9, 8, 5)
    q = T.query("house")
    order = O.oracle_order(q)
    h = U.load(g)
    p = U.plan(q, order, "auto")
    o = M.default_opts(tau_ms=0.0, blocks=1, warps_per_block=1, chunk=8)
    cnt, trace, nt = M.tdfs_test_count_trace(h, p, o)
    assert cnt == O.count(g, q, "auto", order=order)
    assert nt == trace.shape[0] > 0
    two = trace[trace[:, 2] == -2]
    three = trace[trace[:, 2] != -2]
    assert two.shape[0] > 0 and three.shape[0] > 0
    # (a) the first pushes are the first chunk's edges, in directed-edge (CSR) order:
    # the leading run of 2-vertex tasks is strictly increasing in (v1, v2)
    assert trace[0, 2] == -2
    run = int(np.argmax(trace[:, 2] != -2)) if (trace[:, 2] != -2).any() else trace.shape[0]
    keys = trace[:run, 0].astype(np.int64) * g.n + trace[:run, 1]
    assert run >= 1 and (np.diff(keys) > 0).all()
    # (c) 3-prefixes admissible: compare with the oracle's level-2 prefixes
    sub_edges = [(a, b) for a, b in q.edges if a in order[:3] and b in order[:3]]
    E = set(map(tuple, g.edges.tolist())) | {(b, a) for a, b in g.edges.tolist()}
    qpos = {u: i for i, u in enumerate(order)}
    for v1, v2, v3 in three[:5000]:
        S = [int(v1), int(v2), int(v3)]
        assert len(set(S)) == 3
        for a, b in sub_edges:
            assert (S[qpos[a]], S[qpos[b]]) in E
    # every pushed task is dequeued exactly once
    _, st = U.count(g, q, "auto", order=order, stats=True, tau_ms=0.0, blocks=1, warps_per_block=1)
    assert st["tasks_enqueued"] == st["tasks_dequeued"] == nt


def test_split_counts_are_tau_invariant_on_skewed_graph():
    g = T.rmat(13, 16, 2)
    q = T.query("diamond")
    ref = U.count(g, q, "auto", tau_ms=None)
    for tau in (0.0, 0.001, 0.05, 10.0):
        cnt, st = U.count(g, q, "auto", tau_ms=tau, stats=True)
        assert cnt == ref
        if tau == 0.0:
            assert st["tasks_enqueued"] > 0 and st["tasks_enqueued"] == st["tasks_dequeued"]


@pytest.mark.parametrize("range_split", [True, False])
def test_level2_range_tasks_k4(range_split):
    """k = 4: a timed-out level-2 list is split into <= 32 id-range tasks <S0, S1, lo, hi>
     instead of one task per sibling.  With tau = 0 every level-2
    step splits; counts, per-level node counts and W (STATS variant) still equal the
    oracle's, and every pushed task is dequeued exactly once."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    fl = 0 if range_split else M.TDFS_RUN_NO_RANGE_TASKS
    g = T.rmat(11, 12, 4)
    for name in ("c4", "diamond", "k4", "tailed_triangle"):
        q = T.query(name)
        order = O.oracle_order(q)
        r = O.match(g, q, "auto", order=order, deg_filter=True, threads=8)
        for kw in (dict(tau_ms=0.0, flags=fl), dict(tau_ms=0.0, blocks=2, warps_per_block=2, flags=fl),
                   dict(tau_ms=0.01, flags=fl)):
            cnt, st = U.count(g, q, "auto", order=order, stats=True, **kw)
            assert cnt == r["count"], (name, kw)
            assert st["nodes_per_level"][1:q.k] == r["nodes"][1:q.k], (name, kw)
            assert st["adj_bytes"] == r["W"] and st["stream_bytes"] == r["W_stream"], (name, kw)
            assert st["tasks_enqueued"] == st["tasks_dequeued"], (name, kw)
            assert U.count(g, q, "auto", order=order, **kw) == r["count"], (name, kw)
        assert st["tasks_enqueued"] > 0


def test_array_stacks_ablation_same_results():
    """NEXT-4 / E10: array-based stacks (every warp-level owns d_max ids up front, the paper's
    baseline of Tables V-VIII) give the same counts and node counts as paged stacks, and
    their pool is exactly n_warps x levels x E pages."""
    g = T.rmat(11, 12, 4)
    for name in ("c4", "diamond", "house", "c5", "prism"):
        q = T.query(name)
        ref = O.count(g, q, "auto", threads=8)
        for kw in (dict(), dict(tau_ms=0.0), dict(page_bytes=128)):
            cnt, st = U.count(g, q, "auto", stats=True, flags=M.TDFS_RUN_ARRAY_STACKS, **kw)
            assert cnt == ref, (name, kw)
            assert st["pages_used"] == st["pool_pages"] == (
                st["grid_blocks"] * st["warps_per_block"] * (q.k - 3) * st["page_table_entries"]), (name, kw)
            assert U.count(g, q, "auto", flags=M.TDFS_RUN_ARRAY_STACKS, **kw) == ref
