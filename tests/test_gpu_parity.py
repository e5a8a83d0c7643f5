"""Parity of the CUDA path (through the C-ABI) with the CPU oracle, element by element.

Counts and enumerated match sets are integer results: the bar is bit-exact equality.
Sizes: small graphs the oracle finishes in seconds but which still span many warps,
many 32-wide batches, ragged chunk tails, multi-page stack levels (tiny pages), and the
timeout/queue path (tau = 0); then BASELINE.json's full-size configs on sampled shards
(the oracle restricted to the same directed root edges) and closed forms at full size.
"""
import math
import os

import numpy as np
import pytest

import oracle as O
import tdfs_inputs as T
from tests import golden_io as G
from tests import gpu_util as U

pytestmark = pytest.mark.gpu

THREADS = max(1, min(64, os.cpu_count() or 1))

ALL_Q = ["edge", "wedge", "triangle", "path3", "star3", "c4", "diamond", "tailed_triangle", "k4", "house", "c5",
         "k5", "fig1_q", "prism", "w5", "c6", "k6", "k6_minus_e", "w6", "two_k4", "k7", "c8", "k8_minus_e"]


# ------------------------------------------------------------------ Fig. 1
def test_fig1_worked_example():
    d = G.read("fig1.txt")
    g = T.fig1_data()
    q = T.query("fig1_q")
    for cons, key in (([], "M_none"), ([(0, 2)], "M_u1_lt_u3"), ("auto", "M_auto")):
        t, total, ovf = U.enumerate_sorted(g, q, cons if cons != [] else "none")
        assert not ovf
        assert sorted(tuple(int(x) + 1 for x in r) for r in t) == sorted(G.tuples(d[key]))
    assert U.count(g, q, [(0, 2)]) == 2


# ------------------------------------------------------------------ config 1
@pytest.mark.parametrize("m", [10_000, 30_000])
def test_config1_er_fig1_query(m):
    g = T.erdos_renyi(2000, m, 1)
    q = T.query("fig1_q")
    for cons in ([(0, 2)], "auto", "none"):
        assert U.count(g, q, cons) == O.count(g, q, cons), cons
    t, total, _ = U.enumerate_sorted(g, q, [(0, 2)])
    assert np.array_equal(t, O.enumerate_sorted(g, q, [(0, 2)]))


def test_config1_planted():
    g = T.plant(T.erdos_renyi(2000, 10_000, 1), T.fig1_data(), seed=5)
    q = T.query("fig1_q")
    ref = O.count(g, q, [(0, 2)])
    assert ref >= 2
    assert U.count(g, q, [(0, 2)]) == ref
    assert U.count(g, q, "auto") == O.count(g, q, "auto")


# --------------------------------------------------------- all queries, mid graphs
# graphs chosen per query so that the oracle finishes in seconds while the GPU still runs
# thousands of warps, many 32-wide batches and multi-page levels
_GRAPHS = {}


def graph(key):
    if key not in _GRAPHS:
        _GRAPHS[key] = {"r12": lambda: T.rmat(12, 8, 3), "r10": lambda: T.rmat(10, 6, 3),
                        "r9": lambda: T.rmat(9, 5, 3), "er300": lambda: T.erdos_renyi(300, 900, 4),
                        "er400": lambda: T.erdos_renyi(400, 6000, 4)}[key]()
    return _GRAPHS[key]


_ORACLE = {}


def oracle_count(gkey, q, cons="auto", **kw):
    key = (gkey, q.name, str(cons), str(sorted(kw.items())))
    if key not in _ORACLE:
        _ORACLE[key] = O.count(graph(gkey), q, cons, threads=THREADS, **kw)
    return _ORACLE[key]


QUERY_GRAPH = {"edge": "r12", "wedge": "r12", "triangle": "r12", "path3": "r12", "star3": "r12", "c4": "r12",
               "diamond": "r12", "tailed_triangle": "r12", "k4": "r12", "k5": "r12", "house": "r10", "c5": "r10",
               "fig1_q": "r10", "prism": "r10", "w5": "r10", "c6": "r9", "k6": "r9", "k6_minus_e": "r9",
               "w6": "r9", "two_k4": "r9", "k7": "r9", "c8": "er300", "k8_minus_e": "r9"}


@pytest.fixture(scope="module")
def rmat12():
    return graph("r12")


@pytest.mark.parametrize("name", ALL_Q)
def test_counts_all_queries(name):
    q = T.query(name)
    gk = QUERY_GRAPH[name]
    assert U.count(graph(gk), q, "auto") == oracle_count(gk, q, "auto")
    if q.k <= 4 or gk == "er300":
        assert U.count(graph(gk), q, "none") == oracle_count(gk, q, "none")


@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "k4", "house", "c5", "k5", "fig1_q", "prism", "w5"])
def test_counts_dense_er(name):
    q = T.query(name)
    assert U.count(graph("er400"), q, "auto") == oracle_count("er400", q, "auto")


@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "house", "fig1_q", "k5", "prism"])
def test_enumerate_sets(name):
    q = T.query(name)
    g = T.rmat(10, 8, 7) if q.k <= 4 else graph("r9")
    t, total, ovf = U.enumerate_sorted(g, q, "auto")
    ref = O.enumerate_sorted(g, q, "auto")
    assert not ovf and total == ref.shape[0]
    assert np.array_equal(t, ref)


@pytest.mark.parametrize("name,chunk_cap", [("house", 40000), ("diamond", 1500), ("c4", 700), ("triangle", 60)])
def test_enumerate_chunks_stream_every_match_once(name, chunk_cap):
    """NEXT-2: chunked enumeration over refined round-robin sub-shards yields exactly the
    oracle's match set, every chunk within chunk_cap (several chunks per query), also for
    the shards of a 2-rank job."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    q = T.query(name)
    g = T.rmat(7, 4, 3)  # house 124,378 / diamond 5,201 / c4 4,686 / triangle 476 matches
    h = U.load(g)
    p = U.plan(q)
    ref = O.enumerate_sorted(g, q, "auto")
    assert ref.shape[0] > 2 * chunk_cap

    def collect(opts=None):
        chunks = list(M.tdfs_enumerate_chunks(h, p, chunk_cap, opts))
        assert all(0 < c.shape[0] <= chunk_cap for c, _ in chunks)
        return np.concatenate([c for c, _ in chunks]) if chunks else np.zeros((0, q.k), np.int32)

    def srt(t):
        return t[np.lexsort(t.T[::-1])] if t.shape[0] else t

    assert np.array_equal(srt(collect()), ref)
    parts = [collect(M.default_opts(shard_rank=r, shard_world=2)) for r in range(2)]
    assert np.array_equal(srt(np.concatenate(parts)), ref)


@pytest.mark.parametrize("name,ring_cap", [("house", 8), ("house", 4096), ("c4", 64), ("k5", 8), ("edge", 16)])
def test_enumerate_stream_tiny_ring_exact_set(name, ring_cap):
    """NEXT-2 streaming enumerate: a ring far smaller than the output (warps wait for the host to
    drain chunks, many wraps) still delivers exactly the oracle's match set, each match once."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    q = T.query(name)
    g = T.rmat(8, 5, 4)
    h = U.load(g)
    ref = O.enumerate_sorted(g, q, "auto")
    assert ref.shape[0] > 4 * ring_cap
    parts = []
    total = M.tdfs_enumerate_stream(h, U.plan(q), lambda a: parts.append(a), ring_cap,
                                    M.default_opts(tau_ms=0.05))
    got = np.concatenate(parts)
    assert total == ref.shape[0] == got.shape[0]
    assert np.array_equal(got[np.lexsort(got.T[::-1])], ref)
    # a sink that stops early: the call reports it, the job still finishes
    with pytest.raises(M.TdfsError):
        M.tdfs_enumerate_stream(h, U.plan(q), lambda a: True, ring_cap)


def test_enumerate_to_rank_local_files_config2_triangle(c2, tmp_path):
    """NEXT-2 at scale: all 82.7 M triangles of config 2 streamed through a 2^20-tuple ring into two
    rank-local files (shards 0 and 1 of 2); the union has the oracle golden's size, every row is a
    triangle with f(u0) < f(u1) < f(u2) (C_auto) and no row repeats."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    gold = int(G.read("c2_counts.txt")["triangle"].split()[0])
    h = U.load(c2)
    p = M.plan_from_query(T.query("triangle"))
    rows = []
    for r in range(2):
        path = str(tmp_path / f"tri_rank{r}.bin")
        n = M.tdfs_enumerate_to_file(h, p, path, 1 << 20, M.default_opts(shard_rank=r, shard_world=2))
        t = np.fromfile(path, dtype=np.int32).reshape(-1, 3)
        assert t.shape[0] == n
        rows.append(t)
    t = np.concatenate(rows)
    assert t.shape[0] == gold
    assert (t[:, 0] < t[:, 1]).all() and (t[:, 1] < t[:, 2]).all()
    offs, adj = T.to_csr(c2)
    src = np.arange(c2.n, dtype=np.int64).repeat(np.diff(offs))
    key = (src << 32) | adj.astype(np.int64)  # directed edge keys, sorted (CSR order)
    for a, b in ((0, 1), (0, 2), (1, 2)):
        kk = t[:, a].astype(np.int64) << 32 | t[:, b]
        pos = np.searchsorted(key, kk)
        assert (key[np.minimum(pos, key.shape[0] - 1)] == kk).all()
    packed = (t[:, 0].astype(np.int64) << 36) | (t[:, 1].astype(np.int64) << 18) | t[:, 2]
    assert np.unique(packed).shape[0] == gold


def _degree_relabel(g):
    """The (degree, id) ranking of DESIGN.md R35, computed here independently: returns the graph in
    rank ids and orig (rank -> user id)."""
    deg = np.bincount(g.edges.reshape(-1), minlength=g.n)
    orig = np.lexsort((np.arange(g.n), deg))
    rank = np.empty(g.n, dtype=np.int64)
    rank[orig] = np.arange(g.n)
    e = rank[g.edges.astype(np.int64)]
    e = np.sort(e, axis=1)
    lab = None if g.labels is None else g.labels[orig]
    return T.Graph(g.n, e[np.lexsort((e[:, 1], e[:, 0]))].astype(np.int32), lab, g.name + "+deg"), orig


@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "tailed_triangle", "k4", "house", "c5", "k5", "prism",
                                  "w5", "fig1_q"])
def test_degree_order_counts_and_sets(name):
    """TDFS_GRAPH_DEGREE_ORDER (R35): symmetry breaking by degree rank.  Counts equal the oracle's on the
    user graph (any total order picks one embedding per copy); the enumerated tuples, mapped back to user
    ids by the library, equal the oracle's tuples on the rank-relabelled graph mapped back the same way."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    q = T.query(name)
    g = T.rmat(10, 6, 11) if q.k <= 4 else graph("r9")
    h = M.tdfs_load_edges(g.n, g.edges, degree_order=True)
    p = U.plan(q)
    ref = O.count(g, q, "auto", threads=THREADS)
    assert M.tdfs_count(h, p) == ref
    assert M.tdfs_count(h, p, M.default_opts(tau_ms=0.0, page_bytes=128)) == ref
    gr, orig = _degree_relabel(g)
    want = O.enumerate_sorted(gr, q, "auto")
    want = orig[want] if want.shape[0] else want
    want = want[np.lexsort(want.T[::-1])]
    t, total, ovf = M.tdfs_enumerate(h, p, max(ref, 1))
    assert total == ref and not ovf
    t = t[np.lexsort(t.T[::-1])]
    assert np.array_equal(t, want)
    h.free()


def test_enumerate_overflow_keeps_exact_total():
    g = T.rmat(10, 8, 7)
    q = T.query("triangle")
    ref = O.count(g, q, "auto")
    assert ref > 100
    t, total, ovf = U.enumerate_sorted(g, q, "auto", cap=50)
    assert ovf and total == ref and t.shape[0] == 50
    E = set(map(tuple, g.edges.tolist()))
    for r in t:
        a, b, c = sorted(int(x) for x in r)
        assert (a, b) in E and (a, c) in E and (b, c) in E


# ------------------------------------------------------- settings must not change results
@pytest.mark.parametrize("tau_ms", [None, 10.0, 0.0])
@pytest.mark.parametrize("page_bytes", [8192, 128])
def test_tau_and_page_invariance(tau_ms, page_bytes):
    for name in ["diamond", "house", "fig1_q", "c5", "prism"]:
        q = T.query(name)
        ref = oracle_count("r10", q, "auto")
        got = U.count(graph("r10"), q, "auto", tau_ms=tau_ms, page_bytes=page_bytes)
        assert got == ref, (name, tau_ms, page_bytes)


@pytest.mark.parametrize("flags", [0, 4, 8, 12])
def test_reuse_and_shortcut_invariance(flags):
    """Set-intersection result reuse and the count-only last level never
    change results: counts and per-level node counts equal the oracle with every flag combination."""
    g = graph("r10")
    for name in ["k4", "diamond", "tailed_triangle", "house", "k5", "prism", "w5", "fig1_q", "wedge", "star3"]:
        q = T.query(name)
        order = O.oracle_order(q)
        cnt, st = U.count(g, q, "auto", order=order, stats=True, flags=flags)
        r = O.match(g, q, "auto", order=order, deg_filter=True, threads=THREADS)
        assert cnt == r["count"], (name, flags)
        assert st["nodes_per_level"][1:q.k] == r["nodes"][1:q.k], (name, flags)
        assert U.count(g, q, "auto", flags=flags) == r["count"], (name, flags)
    for name in ["k4", "diamond", "two_k4"]:
        q = T.labeled_query(name, 2)
        gl = graph("r10").with_labels(2, 5)
        assert U.count(gl, q, "auto", flags=flags) == O.count(gl, q, "auto", threads=THREADS), (name, flags)


def test_hub_bitmaps_do_not_change_results():
    """Hub adjacency bitmaps (degree >= 256) replace binary searches; results are identical."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    g = T.rmat(12, 24, 5)
    assert int(np.bincount(g.edges.reshape(-1)).max()) >= 256
    # c4: referenced leaf sets F of hubs probed by bitmap against hub leaves (flat leaf batches, streams A/B)
    for name in ["triangle", "k4", "c4"]:
        q = T.query(name)
        ref = O.count(g, q, "auto", threads=THREADS)
        assert U.count(g, q, "auto") == ref
        assert U.count(g, q, "auto", flags=M.TDFS_RUN_NO_HUB_BITMAP) == ref
    for name in ["c4", "diamond", "tailed_triangle", "house"]:
        q = T.query(name)
        assert U.count(g, q, "auto") == U.count(g, q, "auto", flags=M.TDFS_RUN_NO_HUB_BITMAP | 4 | 8), name


def test_leaf_set_paths_do_not_change_results():
    """The staged leaf set F is referenced in place when its list
    has a hub bitmap, materialised in shared memory otherwise, and -- when a materialised F
    would exceed the 512-id stage -- replaced by Eq. (1) per leaf.  The same graph loaded with
    hub bitmaps (default), without (hub_bitmap_bytes = -1: every F materialised, lists of
    degree > 512 take the fallback) and with a 1-hub budget gives the oracle's counts for every
    query shape whose last position is leaf-staged, with the leaf stage on and off."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    g = T.rmat(11, 24, 6)
    deg = np.bincount(g.edges.reshape(-1), minlength=g.n)
    assert int(deg.max()) > 512 and int((deg >= 256).sum()) >= 8  # hubs, and F above the stage
    names = ["c4", "diamond", "tailed_triangle", "k4", "house", "c5"]
    ref = {n: O.count(g, T.query(n), "auto", threads=THREADS) for n in names}
    words = (g.n + 31) // 32
    for hub_bytes in (0, -1, 4 * words):
        h = M.tdfs_load_edges(g.n, g.edges, hub_bitmap_bytes=hub_bytes)
        for n in names:
            p = M.plan_from_query(T.query(n))
            for fl in (0, M.TDFS_RUN_NO_LEAF_STAGE, M.TDFS_RUN_NO_REUSE):
                assert M.tdfs_count(h, p, M.default_opts(flags=fl)) == ref[n], (n, hub_bytes, fl)
        h.free()


def test_chunk_queue_grid_invariance():
    rmat12 = graph("r10")
    q = T.query("house")
    ref = oracle_count("r10", q, "auto")
    for kw in (dict(chunk=1), dict(chunk=32), dict(chunk=7, tau_ms=0.0, queue_ints=30),
               dict(blocks=1, warps_per_block=1, tau_ms=0.0), dict(blocks=3, warps_per_block=2, tau_ms=0.0),
               dict(tau_ms=0.0, queue_ints=3)):
        assert U.count(rmat12, q, "auto", **kw) == ref, kw


def test_order_independence():
    import random
    rng = random.Random(3)
    rmat12 = graph("r10")
    for name in ["diamond", "house", "fig1_q", "prism"]:
        q = T.query(name)
        ref = oracle_count("r10", q, "auto")
        adj = {(a, b) for a, b in q.edges} | {(b, a) for a, b in q.edges}
        for _ in range(3):
            # random connected order
            order = [rng.randrange(q.k)]
            while len(order) < q.k:
                cand = [u for u in range(q.k) if u not in order and any((u, w) in adj for w in order)]
                order.append(rng.choice(cand))
            assert U.count(rmat12, q, "auto", order=order) == ref, (name, order)


def test_shard_sum():
    """Shard-sum invariant for both partitions of the initial edges."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    rmat12 = graph("r10")
    for name in ["triangle", "diamond", "house"]:
        q = T.query(name)
        ref = oracle_count("r10", q, "auto")
        for pol in (M.TDFS_SHARD_ROUND_ROBIN, M.TDFS_SHARD_DEGREE_BALANCED, M.TDFS_SHARD_BLOCKED):
            for W in (2, 3, 8):
                assert sum(U.count(rmat12, q, "auto", shard_rank=r, shard_world=W, shard_policy=pol)
                           for r in range(W)) == ref, (name, pol, W)


@pytest.mark.parametrize("policy", [1, 2])
def test_partitioned_shards_match_oracle_on_owned_edges(policy):
    """A degree-balanced (1) or blocked (2) shard counts exactly the matches whose root edge it owns:
    the oracle restricted to one round-robin shard of W' = nnz (a single edge) summed over the edges
    tdfs_partition_edges gives rank r equals the kernel's rank-r count (small graph, several blocks)."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    g = T.rmat(8, 6, 5)
    offs, adj = T.to_csr(g)
    assert adj.shape[0] > 2 * M.TDFS_SHARD_BLOCK_EDGES
    W = 3
    own = M.tdfs_partition_edges(offs, adj, W, policy)
    q = T.query("diamond")
    order = O.oracle_order(q)
    nnz = adj.shape[0]
    og = O.OracleGraph(g)
    per_edge = [O.count(og, q, "auto", order=order, shard=(e, nnz)) for e in range(nnz)]
    for r in range(W):
        want = sum(c for c, o in zip(per_edge, own) if o == r)
        got = U.count(g, q, "auto", order=order, shard_rank=r, shard_world=W, shard_policy=policy)
        assert got == want, r


def test_labeled_queries():
    g = T.chung_lu(20_000, 120_000, 2.2, 600.0, 7).with_labels(8, 11)
    for name in ["triangle", "c4", "house", "prism", "w5", "w6", "two_k4"]:
        for nl in (8, 2):
            q = T.labeled_query(name, nl)
            assert U.count(g, q, "auto") == O.count(g, q, "auto", threads=THREADS), (name, nl)
    # a single label equals unlabeled
    g1 = T.Graph(g.n, g.edges, np.zeros(g.n, np.uint8), "one-label")
    q = T.query("house")
    assert U.count(g1, q.with_labels([0] * q.k), "auto") == O.count(g1, q, "auto", threads=THREADS)


# ------------------------------------------------------------------ stats parity
@pytest.mark.parametrize("name", ["triangle", "diamond", "house", "fig1_q", "prism"])
def test_nodes_per_level_and_W_match_oracle(name):
    rmat12 = graph("r10")
    q = T.query(name)
    order = O.oracle_order(q)
    for tau in (None, 0.0):
        cnt, st = U.count(rmat12, q, "auto", order=order, stats=True, tau_ms=tau)
        r = O.match(rmat12, q, "auto", order=order, deg_filter=True, threads=THREADS)
        assert cnt == r["count"]
        assert st["nodes_per_level"][1:q.k] == r["nodes"][1:q.k]
        assert st["adj_bytes"] == r["W"]
        assert st["stream_bytes"] == r["W_stream"]


def test_stack_exhaustion_is_an_error_never_a_count():
    import paper_conf_icde_yuan0ha0024_b200 as M
    g = T.rmat(12, 8, 3)
    q = T.query("house")
    with pytest.raises(M.TdfsError) as e:
        U.count(g, q, "auto", page_bytes=128, pool_bytes=128 * 4)
    assert e.value.status == M.TDFS_E_STACK_EXHAUSTED
    with pytest.raises(M.TdfsError) as e:
        U.count(g, q, "auto", page_bytes=128, page_table_entries=1)
    assert e.value.status == M.TDFS_E_STACK_EXHAUSTED


# ------------------------------------------------------------------ edge cases
def test_edge_cases():
    import paper_conf_icde_yuan0ha0024_b200 as M
    empty = T.Graph(10, np.zeros((0, 2), np.int32), None, "empty")
    assert U.count(empty, T.query("triangle"), "auto") == 0
    one = T.from_edge_list(3, [(0, 1)])
    assert U.count(one, T.query("edge"), "auto") == 1
    assert U.count(one, T.query("edge"), "none") == 2
    assert U.count(one, T.query("triangle"), "auto") == 0
    K = T.complete(9)
    for k in range(3, 9):
        assert U.count(K, T.query("triangle" if k == 3 else f"k{k}"), "auto") == math.comb(9, k)
    assert U.count(K, T.query("c4"), "none") == math.perm(9, 4)
    # labels that do not occur
    g = T.rmat(8, 8, 1).with_labels(2, 3)
    q = T.query("triangle").with_labels([5, 5, 5])
    assert U.count(g, q, "auto") == 0
    # contradictory constraints give 0, never an error
    assert U.count(K, T.query("triangle"), [(0, 1), (1, 0)]) == 0
    # duplicate / reversed / self-loop edges in the input are normalised
    h = M.tdfs_load_edges(4, np.array([[0, 1], [1, 0], [1, 2], [2, 2], [2, 0], [0, 1]]))
    p = M.plan_from_query(T.query("triangle"))
    assert M.tdfs_count(h, p) == 1
    assert h.info()["m"] == 3


def test_invalid_csr_rejected():
    import paper_conf_icde_yuan0ha0024_b200 as M
    offs = np.array([0, 2, 3, 4], np.int64)
    adj = np.array([2, 1, 0, 0], np.int32)  # unsorted list of vertex 0
    with pytest.raises(M.TdfsError) as e:
        M.tdfs_load_graph(offs, adj, validate=True)
    assert e.value.status == M.TDFS_E_GRAPH_FORMAT
    h = M.tdfs_load_graph(offs, adj, normalize=True)
    assert h.info()["m"] == 2
    bad = np.array([0, 1, 2, 2], np.int64)
    with pytest.raises(M.TdfsError) as e:
        M.tdfs_load_graph(bad, np.array([7, 0], np.int32), validate=True)
    assert e.value.status in (M.TDFS_E_GRAPH_FORMAT, M.TDFS_E_ID_RANGE)


def _numpy_csr(g):
    """Input-format conversion for the DEVICE_BORROW test (plain numpy, no matching)."""
    a = np.concatenate([g.edges[:, 0], g.edges[:, 1]]).astype(np.int64)
    b = np.concatenate([g.edges[:, 1], g.edges[:, 0]]).astype(np.int64)
    idx = np.lexsort((b, a))
    offs = np.zeros(g.n + 1, np.int64)
    np.add.at(offs, a + 1, 1)
    return np.cumsum(offs), b[idx].astype(np.int32)


def test_device_borrow_csr():
    import torch
    import paper_conf_icde_yuan0ha0024_b200 as M
    g = T.rmat(10, 8, 9)
    offs, adj = _numpy_csr(g)
    to = torch.from_numpy(offs).cuda()
    ta = torch.from_numpy(adj).cuda()
    hb = M.tdfs_load_graph(to, ta, validate=True)
    assert hb.info()["m"] == g.m
    p = M.plan_from_query(T.query("diamond"))
    assert M.tdfs_count(hb, p) == O.count(g, T.query("diamond"), "auto")
    bad = ta.clone()
    bad[0], bad[1] = ta[1], ta[0]  # break the order of the first list
    with pytest.raises(M.TdfsError):
        M.tdfs_load_graph(to, bad, validate=True)


# ------------------------------------------------------------------ full-size configs
@pytest.fixture(scope="module")
def c2():
    return T.config_graph(2)


def test_config2_full_triangle_and_closed_forms(c2):
    q = T.query("triangle")
    assert U.count(c2, q, "auto") == O.count(c2, q, "auto", threads=THREADS)
    d = np.bincount(c2.edges.reshape(-1), minlength=c2.n).astype(object)
    assert U.count(c2, T.query("wedge"), "auto") == int(sum(x * (x - 1) // 2 for x in d))
    assert U.count(c2, T.query("star3"), "auto") == int(sum(x * (x - 1) * (x - 2) // 6 for x in d))


@pytest.mark.parametrize("name", ["c4", "diamond", "tailed_triangle", "k4"])
def test_config2_full_sampled_shards(c2, name):
    """Full C2 graph in the bench launch configuration; the oracle computes the matches
    rooted at the sampled shard's directed edges (same order, so the same root edges)."""
    q = T.query(name)
    order = O.oracle_order(q)
    W = 4001
    for r in (0, 1777):
        got = U.count(c2, q, "auto", order=order, shard_rank=r, shard_world=W)
        ref = O.count(c2, q, "auto", order=order, shard=(r, W), threads=THREADS)
        assert got == ref, (name, r)


def test_config2_full_counts_equal_oracle_goldens(c2):
    """The five benched C2 counts, in bench.py's launch configuration (planner order, tau = 10 ms,
    chunk 8 / 1), equal the oracle's full-graph counts, written to tests/golden/c2_counts.txt by
    scripts/golden_counts.py (oracle/ only; M is order-independent, R9)."""
    import paper_conf_icde_yuan0ha0024_b200 as M
    gold = {k: int(v.split()[0]) for k, v in G.read("c2_counts.txt").items()}
    assert set(gold) >= set(T.CONFIG_QUERIES[2])
    h = U.load(c2)
    for name in T.CONFIG_QUERIES[2]:
        q = T.query(name)
        o = M.default_opts(chunk=8 if q.k <= 3 else 1)
        assert M.tdfs_count(h, M.plan_from_query(q), o) == gold[name], name
        if name != "triangle":  # and the oracle-order plan whose shards are checked above
            assert U.count(c2, q, "auto", order=O.oracle_order(q)) == gold[name], name
