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
def _level2_candidates(g, q, order, cons, v1, v2):
    """Admissible f(pi_2) after the prefix (v1, v2), from the definition (sorted): adjacent to
    the matched backward neighbours, distinct, inside the constraint window, degree filter of
    DESIGN.md R8 (deg_Q(pi_2) > |B(pi_2)|)."""
    nb = [set() for _ in range(g.n)]
    for a, b in g.edges.tolist():
        nb[a].add(b)
        nb[b].add(a)
    qadj = {(a, b) for a, b in q.edges} | {(b, a) for a, b in q.edges}
    u = order[2]
    S = [v1, v2]
    back = [j for j in range(2) if (order[j], u) in qadj]
    cand = set(range(g.n))
    for j in back:
        cand &= nb[S[j]]
    cand -= {v1, v2}
    pos = {w: i for i, w in enumerate(order)}
    for a, b in cons:  # f(a) < f(b)
        if pos[b] == 2 and pos[a] < 2:
            cand = {x for x in cand if x > S[pos[a]]}
        if pos[a] == 2 and pos[b] < 2:
            cand = {x for x in cand if x < S[pos[b]]}
    dq = sum(1 for a, b in q.edges if u in (a, b))
    if dq > len(back):
        cand = {x for x in cand if len(nb[x]) >= dq}
    return sorted(cand)


def test_timeout_split_single_warp_trace():
    """Fig. 5 / Alg. 4 exactly, tau = 0, one warp, the paper's split rule
    (TDFS_RUN_NO_RANGE_TASKS): the warp takes a chunk of 8 directed edges and, timing out before
    the first descent, pushes the chunk's filtered-in edges as <v1, v2, -2> in CSR order; it then
    dequeues them in FIFO order and, timing out at level 2 of each, pushes the current candidate and
    all its siblings <v1, v2, v3> in ascending order; 3-prefix tasks (<= 3 matched vertices) are
    never split further; then the next chunk.  The whole trace is derived from the definition."""
    g = T.rmat(8, 6, 5)
    q = T.query("house")
    order = O.oracle_order(q)
    cons = O.automorphisms(q)[1]
    h = U.load(g)
    p = U.plan(q, order, "auto")
    o = M.default_opts(tau_ms=0.0, blocks=1, warps_per_block=1, chunk=8, flags=M.TDFS_RUN_NO_RANGE_TASKS)
    cnt, trace, nt = M.tdfs_test_count_trace(h, p, o)
    assert cnt == O.count(g, q, "auto", order=order)
    # expected: edge filter of positions 0, 1 (degree >= deg_Q, the (u1, u2) constraint)
    offs, adj = T.to_csr(g)
    deg = np.diff(offs)
    src = np.repeat(np.arange(g.n), deg)
    dq = [sum(1 for a, b in q.edges if u in (a, b)) for u in range(q.k)]
    c01 = [(a, b) for a, b in cons if {a, b} == {order[0], order[1]}]
    want = []
    for c0 in range(0, adj.shape[0], 8):
        edges = []
        for e in range(c0, min(c0 + 8, adj.shape[0])):
            v1, v2 = int(src[e]), int(adj[e])
            if deg[v1] < dq[order[0]] or deg[v2] < dq[order[1]]:
                continue
            if any((a == order[0] and not v1 < v2) or (a == order[1] and not v2 < v1) for a, b in c01):
                continue
            edges.append((v1, v2))
        want += [(v1, v2, -2) for v1, v2 in edges]
        for v1, v2 in edges:
            want += [(v1, v2, x) for x in _level2_candidates(g, q, order, cons, v1, v2)]
    got = [tuple(int(x) for x in r) for r in trace]
    assert nt == len(want)
    assert got == want
    # every pushed task is dequeued exactly once
    _, st = U.count(g, q, "auto", order=order, stats=True, tau_ms=0.0, blocks=1, warps_per_block=1,
                    flags=M.TDFS_RUN_NO_RANGE_TASKS)
    assert st["tasks_enqueued"] == st["tasks_dequeued"] == nt


def test_deep_range_tasks_tau_zero():
    """R33: with range tasks on (default) a timed-out level d (2 <= d <= min(4, k-2)) is split into
    <= 32 id-range tasks <S0..S_{d-1}, lo, hi>; tau = 0 splits at every eligible step.  Counts,
    per-level node counts and roofline bytes (STATS) still equal the oracle's for k = 5..7, every
    pushed task is dequeued exactly once, and the trace shows range tasks at levels 3 and 4."""
    g = T.rmat(8, 6, 8)  # w6: 18.5 M matches, 7.3 M level-5 prefixes
    for name in ("house", "c5", "k5", "prism", "w6"):
        q = T.query(name)
        order = O.oracle_order(q)
        r = O.match(g, q, "auto", order=order, deg_filter=True, threads=8)
        for kw in (dict(tau_ms=0.0), dict(tau_ms=0.0, blocks=2, warps_per_block=2), dict(tau_ms=0.002)):
            cnt, st = U.count(g, q, "auto", order=order, stats=True, **kw)
            assert cnt == r["count"], (name, kw)
            assert st["nodes_per_level"][1:q.k] == r["nodes"][1:q.k], (name, kw)
            assert st["stream_bytes"] == r["W_stream"], (name, kw)
            assert st["tasks_enqueued"] == st["tasks_dequeued"], (name, kw)
            assert U.count(g, q, "auto", order=order, **kw) == r["count"], (name, kw)
    q = T.query("w6")
    h = U.load(g)
    cnt, trace, nt = M.tdfs_test_count_trace(h, U.plan(q, O.oracle_order(q), "auto"),
                                             M.default_opts(tau_ms=0.0, blocks=2, warps_per_block=2))
    kinds = set(int(x) for x in trace[:, 2] if x < -2)
    assert {-5, -6} <= kinds, kinds  # range tasks at levels 2 (-5), 3 (-6) and 4 (-7)


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
