"""Pins for the CPU oracle (no GPU).  Each test ties the oracle to something other than
itself: the paper's Fig. 1 worked example, closed forms, textbook automorphism group
orders, brute force (O1), networkx VF2 (O3) and networkx triangle / clique routines.
"""
import itertools
import math
import random

import numpy as np
import pytest

import oracle as O
import tdfs_inputs as T
from tests import golden_io as G

# Textbook |Aut| of the standard patterns (dihedral / symmetric groups etc.).
AUT = {"edge": 2, "wedge": 2, "triangle": 6, "path3": 2, "star3": 6, "c4": 8, "diamond": 4,
       "tailed_triangle": 2, "k4": 24, "house": 2, "c5": 10, "k5": 120, "star4": 24, "fig1_q": 4,
       "prism": 12, "w5": 10, "c6": 12, "k6": 720, "k6_minus_e": 48, "w6": 12, "two_k4": 72,
       "k7": 5040, "k7_minus_e": 240, "k8": 40320, "k8_minus_e": 1440, "c8": 16}


def _fig1():
    d = G.read("fig1.txt")
    qe = [(a - 1, b - 1) for a, b in G.pairs(d["query_edges"])]
    de = [(a - 1, b - 1) for a, b in G.pairs(d["data_edges"])]
    return d, T.Query("fig1", 5, qe), T.from_edge_list(7, de, "fig1")


def _rows(arr):
    return sorted(tuple(int(x) + 1 for x in r) for r in arr)


# ------------------------------------------------------------------ Fig. 1
def test_fig1_golden_sets():
    d, q, g = _fig1()
    assert q.edges == T.query("fig1_q").edges and np.array_equal(g.edges, T.fig1_data().edges)
    assert _rows(O.enumerate_sorted(g, q, "none")) == sorted(G.tuples(d["M_none"]))
    assert _rows(O.enumerate_sorted(g, q, [(0, 2)])) == sorted(G.tuples(d["M_u1_lt_u3"]))
    assert _rows(O.enumerate_sorted(g, q, "auto")) == sorted(G.tuples(d["M_auto"]))
    s1 = tuple(G.ints(d["match"]))
    s2 = tuple(G.ints(d["suppressed_by_u1_lt_u3"]))
    assert s1 in _rows(O.enumerate_sorted(g, q, [(0, 2)]))
    assert s2 in _rows(O.enumerate_sorted(g, q, "none"))
    assert s2 not in _rows(O.enumerate_sorted(g, q, [(0, 2)]))


def test_fig1_levels_and_degree_pruning():
    d, q, g = _fig1()
    # level 3 after [v1, v2]: matches of the sub-query on {u1,u2,u3} extending (v1, v2)
    sub = T.Query("tri", 3, [(0, 1), (0, 2), (1, 2)])
    t = O.enumerate_sorted(g, sub, "none")
    lvl3 = sorted(int(r[2]) + 1 for r in t if r[0] == 0 and r[1] == 1)
    assert lvl3 == G.ints(d["level3_after_v1_v2"])
    # level 4 after [v1, v2, v3]: sub-query on {u1..u4}
    sub4 = T.Query("s4", 4, [(0, 1), (0, 2), (1, 2), (0, 3), (2, 3)])
    t4 = O.enumerate_sorted(g, sub4, "none")
    lvl4 = sorted(int(r[3]) + 1 for r in t4 if (r[0], r[1], r[2]) == (0, 1, 2))
    assert lvl4 == G.ints(d["level4_after_v1_v2_v3"])
    # degree pruning at u1: with the filter, only v1..v4 survive position 0
    r = O.match(g, q, "none", order=[0, 1, 2, 3, 4], deg_filter=True)
    pruned = set(G.ints(d["pruned_at_u1"]))
    assert r["nodes"][0] == 7 - len(pruned)
    r0 = O.match(g, q, "none", order=[0, 1, 2, 3, 4], deg_filter=False)
    assert r0["nodes"][0] == 7 and r0["count"] == r["count"] == 4


def test_fig1_aut():
    _, q, _ = _fig1()
    n_aut, cons = O.automorphisms(q)
    assert n_aut == 4
    assert sorted(cons) == [(0, 2), (1, 3)]


# ------------------------------------------------------------ closed forms
@pytest.mark.parametrize("name", sorted(AUT))
def test_aut_orders_textbook(name):
    assert O.automorphisms(T.query(name))[0] == AUT[name]


@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "tailed_triangle", "k4", "house", "c5",
                                  "k5", "fig1_q", "star3", "path3", "prism", "w5", "c6"])
def test_complete_graph_closed_forms(name):
    q = T.query(name)
    n = 7 if q.k <= 6 else 8
    K = T.complete(n)
    inj = math.perm(n, q.k)          # every injective map is an embedding into K_n
    assert O.count(K, q, "none") == inj
    assert O.count(K, q, "auto") * AUT[name] == inj  # copies = C(n,k) k! / |Aut|


@pytest.mark.parametrize("k,n", [(3, 9), (4, 9), (5, 9), (6, 9), (7, 9), (8, 10)])
def test_cliques_in_complete_graph(k, n):
    assert O.count(T.complete(n), T.query(f"k{k}" if k > 3 else "triangle"), "auto") == math.comb(n, k)


@pytest.mark.parametrize("a,b", [(3, 4), (4, 5), (2, 6)])
def test_complete_bipartite(a, b):
    g = T.complete_bipartite(a, b)
    assert O.count(g, T.query("triangle"), "auto") == 0
    assert O.count(g, T.query("c4"), "auto") == math.comb(a, 2) * math.comb(b, 2)
    assert O.count(g, T.query("k4"), "auto") == 0


@pytest.mark.parametrize("r,c", [(3, 4), (4, 5), (6, 6)])
def test_grid(r, c):
    g = T.grid(r, c)
    assert O.count(g, T.query("triangle"), "auto") == 0
    assert O.count(g, T.query("c4"), "auto") == (r - 1) * (c - 1)


def _degrees(g):
    return np.bincount(g.edges.reshape(-1), minlength=g.n).astype(np.int64)


@pytest.mark.parametrize("gen", ["er", "rmat"])
def test_stars_and_wedges_closed_form(gen):
    g = T.erdos_renyi(300, 1500, 3) if gen == "er" else T.rmat(8, 4, 5)
    d = _degrees(g)
    assert O.count(g, T.query("wedge"), "auto") == sum(math.comb(int(x), 2) for x in d)
    assert O.count(g, T.query("star3"), "auto") == sum(math.comb(int(x), 3) for x in d)
    assert O.count(g, T.query("star4"), "auto") == sum(math.comb(int(x), 4) for x in d)
    assert O.count(g, T.query("edge"), "auto") == g.m


def test_path3_closed_form_with_networkx_triangles():
    import networkx as nx
    g = T.rmat(9, 8, 2)
    d = _degrees(g)
    G_ = nx.Graph()
    G_.add_edges_from(map(tuple, g.edges.tolist()))
    tri = sum(nx.triangles(G_).values()) // 3
    # paths with 3 edges = sum over edges (d_u - 1)(d_v - 1) - 3 * triangles
    p3 = int(sum((d[a] - 1) * (d[b] - 1) for a, b in g.edges)) - 3 * tri
    assert O.count(g, T.query("path3"), "auto") == p3
    assert O.count(g, T.query("triangle"), "auto") == tri


def test_cliques_networkx():
    import networkx as nx
    g = T.rmat(8, 10, 4)
    G_ = nx.Graph()
    G_.add_edges_from(map(tuple, g.edges.tolist()))
    by_k = {}
    for c in nx.enumerate_all_cliques(G_):
        by_k[len(c)] = by_k.get(len(c), 0) + 1
    for k in (3, 4, 5, 6):
        name = "triangle" if k == 3 else f"k{k}"
        assert O.count(g, T.query(name), "auto") == by_k.get(k, 0), k


# ------------------------------------------------------------- brute force
SMALL_QUERIES = ["edge", "wedge", "triangle", "path3", "star3", "c4", "diamond", "tailed_triangle", "k4",
                 "house", "c5", "fig1_q", "prism", "w5", "c6", "k6_minus_e", "w6", "two_k4", "c8",
                 "k8_minus_e"]


@pytest.mark.parametrize("name", SMALL_QUERIES)
def test_bruteforce_agreement(name):
    q = T.query(name)
    rng = random.Random(sum(map(ord, name)))
    for trial in range(3):
        n = rng.choice([8, 9, 10]) if q.k <= 6 else rng.choice([8, 9])
        g = T.small_random(n, rng.choice([0.4, 0.6, 0.8]), seed=trial + 17)
        for cons in ("none", "auto", "rand"):
            if cons == "rand":
                pairs = [(a, b) for a in range(q.k) for b in range(q.k) if a != b]
                c = rng.sample(pairs, min(2, len(pairs)))
                c = [p for p in c if (p[1], p[0]) not in c]
            elif cons == "auto":
                c = O.automorphisms(q)[1]
            else:
                c = []
            bf = O.bruteforce(g, q, c)
            o2 = O.enumerate_sorted(g, q, c)
            assert np.array_equal(bf, o2), (name, trial, cons)


def test_bruteforce_labeled():
    rng = random.Random(5)
    for trial in range(6):
        g = T.small_random(10, 0.6, seed=100 + trial)
        g.labels = np.array([rng.randrange(3) for _ in range(g.n)], dtype=np.uint8)
        for name in ["triangle", "c4", "diamond", "house", "fig1_q"]:
            q = T.labeled_query(name, 3)
            c = O.automorphisms(q)[1]
            assert np.array_equal(O.bruteforce(g, q, c), O.enumerate_sorted(g, q, c))
            assert np.array_equal(O.bruteforce(g, q, []), O.enumerate_sorted(g, q, "none"))


# ------------------------------------------------------------------- VF2
@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "tailed_triangle", "k4", "house", "c5",
                                  "fig1_q"])
def test_vf2_agreement(name):
    g = T.erdos_renyi(60, 240, 9)
    q = T.query(name)
    assert O.count(g, q, "none") == O.vf2_count(g, q)


def test_vf2_labeled():
    g = T.erdos_renyi(50, 260, 2).with_labels(2, 3)
    for name in ["triangle", "c4", "house"]:
        q = T.labeled_query(name, 2)
        assert O.count(g, q, "none") == O.vf2_count(g, q)


# -------------------------------------------------------------- invariants
@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "tailed_triangle", "k4", "house", "c5",
                                  "fig1_q", "prism", "w5"])
def test_aut_invariant(name):
    g = T.rmat(8, 6, 7)
    q = T.query(name)
    assert O.count(g, q, "auto") * AUT[name] == O.count(g, q, "none")


def test_order_and_filter_independence():
    g = T.rmat(8, 6, 3)
    rng = random.Random(1)
    for name in ["diamond", "house", "c5", "fig1_q", "prism"]:
        q = T.query(name)
        ref = O.count(g, q, "auto")
        for _ in range(4):
            perm = list(range(q.k))
            rng.shuffle(perm)
            assert O.count(g, q, "auto", order=perm) == ref
            assert O.count(g, q, "auto", order=perm, deg_filter=False) == ref


def test_labels_single_label_and_sum_over_labelings():
    g = T.erdos_renyi(40, 150, 4)
    g1 = T.Graph(g.n, g.edges, np.zeros(g.n, np.uint8), "one-label")
    for name in ["triangle", "c4", "tailed_triangle"]:
        q = T.query(name)
        assert O.count(g1, q.with_labels([0] * q.k), "none") == O.count(g, q, "none")
    g2 = g.with_labels(2, 9)
    for name in ["triangle", "c4"]:
        q = T.query(name)
        tot = sum(O.count(g2, q.with_labels(lab), "none") for lab in itertools.product(range(2), repeat=q.k))
        assert tot == O.count(g, q, "none")


def test_shard_sum():
    g = T.rmat(9, 6, 11)
    for name in ["triangle", "diamond", "house"]:
        q = T.query(name)
        ref = O.count(g, q, "auto")
        for W in (2, 3, 7):
            assert sum(O.count(g, q, "auto", shard=(r, W)) for r in range(W)) == ref


def test_threads_equal_serial():
    g = T.rmat(10, 8, 12)
    q = T.query("c4")
    assert O.count(g, q, "auto", threads=4) == O.count(g, q, "auto", threads=1)


def test_nodes_and_W_triangle_closed_form():
    """Triangle, order [0,1,2], constraints 0<1<2, degree filter on:
    internal prefixes are the edges u<v with deg >= 2 at both ends;
    W = sum over them of 4 (d_u + d_v) + 32 (two operands, 16 B of offsets each)."""
    g = T.rmat(10, 8, 13)
    d = _degrees(g)
    r = O.match(g, T.query("triangle"), "auto", order=[0, 1, 2], deg_filter=True)
    u, v = g.edges[:, 0], g.edges[:, 1]
    ok = (d[u] >= 2) & (d[v] >= 2)
    assert r["nodes"][1] == int(ok.sum())
    assert r["W"] == int((4 * (d[u] + d[v]) + 32)[ok].sum())
    assert r["nodes"][2] == r["count"]


def test_W_stream_triangle_closed_form():
    """R32 roofline bytes for the triangle, order [0,1,2], constraints 0<1<2: each internal
    prefix (edge u<v, both degrees >= 2) adds 2 x 16 B + 4 B x min(|N(u) > v|, |N(v) > v|)
    (no earlier candidate set can be a source at position 2)."""
    g = T.rmat(10, 8, 13)
    d = _degrees(g)
    nbrs = [[] for _ in range(g.n)]
    for a, b in g.edges.tolist():
        nbrs[a].append(b)
        nbrs[b].append(a)
    tot = 0
    for u, v in g.edges.tolist():
        if d[u] >= 2 and d[v] >= 2:
            tot += 32 + 4 * min(sum(1 for w in nbrs[u] if w > v), sum(1 for w in nbrs[v] if w > v))
    assert O.match(g, T.query("triangle"), "auto", order=[0, 1, 2])["W_stream"] == tot
    # a count-only single-operand last position streams nothing: wedge = 16 B per prefix
    r = O.match(g, T.query("wedge"), "auto", order=[0, 1, 2])
    assert r["W_stream"] == 16 * r["nodes"][1]


def test_W_stream_diamond_reuse_closed_form():
    """R32 with a reuse source: diamond in the planner's order [1, 2, 0, 3]
    with C_auto = {u0 < u3, u1 < u2}.  Position 2 (u0, B = {p0, p1}, no window) adds
    32 B + 4 B x min(deg a, deg b) per edge prefix a < b with deg >= 3; position 3 (u3, same
    B, window > S[2]) has C(2) as a source that alone is its candidate set, so it is count-only:
    32 B per prefix (a, b, c), c any common neighbour.  Closed form with numpy (A @ A)."""
    g = T.rmat(9, 8, 17)
    n = g.n
    A = np.zeros((n, n), dtype=np.int64)
    A[g.edges[:, 0], g.edges[:, 1]] = 1
    A[g.edges[:, 1], g.edges[:, 0]] = 1
    d = A.sum(1)
    common = A @ A
    tot = 0
    for a, b in g.edges.tolist():  # a < b (canonical), the edge constraint S0 < S1
        if d[a] >= 3 and d[b] >= 3:
            tot += 32 + 4 * int(min(d[a], d[b])) + 32 * int(common[a, b])
    q = T.query("diamond")
    assert O.automorphisms(q)[1] == [(0, 3), (1, 2)]
    r = O.match(g, q, "auto", order=[1, 2, 0, 3])
    assert r["W_stream"] == tot


def test_enumerate_tuples_satisfy_definition():
    g = T.rmat(8, 6, 21)
    q = T.query("house")
    cons = O.automorphisms(q)[1]
    t = O.enumerate_sorted(g, q, cons)
    assert t.shape[0] == O.count(g, q, cons)
    E = set(map(tuple, g.edges.tolist()))
    for row in t[:2000]:
        assert len(set(row.tolist())) == q.k
        for a, b in q.edges:
            x, y = int(row[a]), int(row[b])
            assert (min(x, y), max(x, y)) in E
        for a, b in cons:
            assert row[a] < row[b]
