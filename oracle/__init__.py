"""TEST INFRASTRUCTURE ONLY -- the CPU oracle for the T-DFS hot path.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (cpu_baseline leg and
``--impl reference``) may import this package.  It shares no code with the product
package ``paper_conf_icde_yuan0ha0024_b200`` and never consumes anything the product
computes.

Three independent oracles:

* O2 ``match`` -- ``oracle.cpp``: Algorithm 1 + Eq. (1) written out literally
  (PAPER.md:54-82), serial (optionally fanned out over root vertices with threads).
* O1 ``bruteforce`` -- generate-and-test over injective maps (no intersections), tiny graphs.
* O3 ``vf2_count`` -- networkx VF2 monomorphisms (a library routine).

Symmetry-breaking constraints: ``automorphisms`` brute-forces Aut(Q) and builds the
stabilizer-chain constraint set (R3).
"""
from __future__ import annotations

import ctypes
import itertools
import os
import subprocess
from typing import Iterable, List, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

I32P = ctypes.POINTER(ctypes.c_int32)
U64P = ctypes.POINTER(ctypes.c_uint64)
I64P = ctypes.POINTER(ctypes.c_int64)
U8P = ctypes.POINTER(ctypes.c_uint8)


def build_oracle(force: bool = False) -> str:
    """Compile oracle.cpp -> liboracle.so with plain g++ (no CUDA, no product headers)."""
    src = os.path.join(_HERE, "oracle.cpp")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-pthread", "-o", tmp, src])
        os.replace(tmp, _SO)
    return _SO


def _o():
    global _lib
    if _lib is None:
        build_oracle()
        lib = ctypes.CDLL(_SO)
        lib.oracle_match.restype = ctypes.c_int
        lib.oracle_match.argtypes = [ctypes.c_int64, ctypes.c_int64, I32P, I32P, U8P,
                                     ctypes.c_int, ctypes.c_int, I32P, I32P,
                                     ctypes.c_int, I32P, I32P, ctypes.c_int,
                                     ctypes.c_int, ctypes.c_int, ctypes.c_int64, ctypes.c_int64,
                                     ctypes.c_int, ctypes.c_int64, I32P,
                                     U64P, U64P, U64P, U64P]
        lib.oracle_graph_new.restype = ctypes.c_void_p
        lib.oracle_graph_new.argtypes = [ctypes.c_int64, ctypes.c_int64, I32P, I32P, U8P]
        lib.oracle_graph_free.restype = None
        lib.oracle_graph_free.argtypes = [ctypes.c_void_p]
        lib.oracle_match_g.restype = ctypes.c_int
        lib.oracle_match_g.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, I32P, I32P,
                                       ctypes.c_int, I32P, I32P, ctypes.c_int,
                                       ctypes.c_int, ctypes.c_int, ctypes.c_int64, ctypes.c_int64,
                                       ctypes.c_int, ctypes.c_int64, I32P,
                                       U64P, U64P, U64P, U64P]
        lib.oracle_order.restype = ctypes.c_int
        lib.oracle_order.argtypes = [ctypes.c_int, ctypes.c_int, I32P, I32P]
        lib.oracle_automorphisms.restype = ctypes.c_int
        lib.oracle_automorphisms.argtypes = [ctypes.c_int, ctypes.c_int, I32P, I32P, I64P, I32P, ctypes.c_int]
        _lib = lib
    return _lib


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def _p(a: Optional[np.ndarray], t):
    return None if a is None else a.ctypes.data_as(t)


def automorphisms(query) -> Tuple[int, List[Tuple[int, int]]]:
    """(|Aut(Q)|, stabilizer-chain constraints [(a, b): f(a) < f(b)])."""
    q = query
    qe = _i32(q.edges).reshape(-1)
    ql = None if q.labels is None else _i32(q.labels)
    n_aut = ctypes.c_int64(0)
    pairs = np.zeros(2 * 64, dtype=np.int32)
    npairs = _o().oracle_automorphisms(q.k, len(q.edges), _p(qe, I32P), _p(ql, I32P), ctypes.byref(n_aut),
                                       _p(pairs, I32P), 64)
    if npairs < 0:
        raise ValueError("bad query")
    return int(n_aut.value), [(int(pairs[2 * i]), int(pairs[2 * i + 1])) for i in range(npairs)]


def oracle_order(query) -> List[int]:
    qe = _i32(query.edges).reshape(-1)
    out = np.zeros(query.k, dtype=np.int32)
    if _o().oracle_order(query.k, len(query.edges), _p(qe, I32P), _p(out, I32P)) != 0:
        raise ValueError("bad query")
    return [int(x) for x in out]


def _constraints(query, constraints) -> List[Tuple[int, int]]:
    if constraints is None or constraints == "none":
        return []
    if constraints == "auto":
        return automorphisms(query)[1]
    return [(int(a), int(b)) for a, b in constraints]


class OracleGraph:
    """The oracle's adjacency built once for many queries (large configs)."""

    def __init__(self, graph):
        self.graph = graph
        g = graph
        eu = _i32(g.edges[:, 0]) if g.m else np.zeros(1, np.int32)
        ev = _i32(g.edges[:, 1]) if g.m else np.zeros(1, np.int32)
        self._lab = None if g.labels is None else np.ascontiguousarray(g.labels, dtype=np.uint8)
        self.ptr = _o().oracle_graph_new(g.n, g.m, _p(eu, I32P), _p(ev, I32P), _p(self._lab, U8P))

    def __del__(self):
        try:
            if self.ptr:
                _o().oracle_graph_free(self.ptr)
                self.ptr = None
        except Exception:
            pass


def match(graph, query, constraints="auto", order: Optional[Sequence[int]] = None, deg_filter: bool = True,
          shard: Tuple[int, int] = (0, 1), roots: Optional[Tuple[int, int]] = None, threads: int = 1,
          enumerate_cap: int = 0):
    """Run O2 on a tdfs_inputs.Graph or an OracleGraph.
    Returns dict(count, nodes (list, k), W, W_stream, tuples (ndarray or None), overflow)."""
    q = query
    qe = _i32(q.edges).reshape(-1)
    ql = None if q.labels is None else _i32(q.labels)
    cons = _constraints(q, constraints)
    ca = _i32(cons).reshape(-1) if cons else np.zeros(2, np.int32)
    oa = None if order is None else _i32(order)
    cnt = ctypes.c_uint64(0)
    nodes = np.zeros(9, dtype=np.uint64)
    w = ctypes.c_uint64(0)
    sb = ctypes.c_uint64(0)
    out = np.zeros(max(1, enumerate_cap) * q.k, dtype=np.int32) if enumerate_cap > 0 else None
    rlo, rhi = (0, -1) if roots is None else roots
    tail = (len(cons), _p(ca, I32P), _p(oa, I32P), int(bool(deg_filter)),
            int(shard[0]), int(shard[1]), int(rlo), int(rhi),
            int(threads), int(enumerate_cap), _p(out, I32P),
            ctypes.byref(cnt), nodes.ctypes.data_as(U64P), ctypes.byref(w), ctypes.byref(sb))
    if isinstance(graph, OracleGraph):
        rc = _o().oracle_match_g(graph.ptr, q.k, len(q.edges), _p(qe, I32P), _p(ql, I32P), *tail)
    else:
        g = graph
        eu = _i32(g.edges[:, 0]) if g.m else np.zeros(1, np.int32)
        ev = _i32(g.edges[:, 1]) if g.m else np.zeros(1, np.int32)
        lab = None if g.labels is None else np.ascontiguousarray(g.labels, dtype=np.uint8)
        rc = _o().oracle_match(g.n, g.m, _p(eu, I32P), _p(ev, I32P), _p(lab, U8P),
                               q.k, len(q.edges), _p(qe, I32P), _p(ql, I32P), *tail)
    if rc < 0:
        raise ValueError("oracle_match: bad arguments")
    res = {"count": int(cnt.value), "nodes": [int(x) for x in nodes[: q.k]], "W": int(w.value),
           "W_stream": int(sb.value), "tuples": None, "overflow": rc == 1}
    if enumerate_cap > 0:
        n = min(res["count"], enumerate_cap)
        res["tuples"] = out[: n * q.k].reshape(n, q.k).copy()
    return res


def count(graph, query, constraints="auto", **kw) -> int:
    return match(graph, query, constraints, **kw)["count"]


def enumerate_sorted(graph, query, constraints="auto", cap: Optional[int] = None, **kw) -> np.ndarray:
    """All tuples (f(u_0), ..., f(u_{k-1})) as a lexicographically sorted (M, k) array."""
    if cap is None:
        cap = match(graph, query, constraints, **kw)["count"]
    if cap == 0:
        return np.zeros((0, query.k), dtype=np.int32)
    t = match(graph, query, constraints, enumerate_cap=cap, **kw)["tuples"]
    return t[np.lexsort(t.T[::-1])]


# --------------------------------------------------------------------- O1
def bruteforce(graph, query, constraints: Iterable[Tuple[int, int]] = ()) -> np.ndarray:
    """Generate-and-test over all injective maps f: V_Q -> V (tiny graphs only).

    Maps are grown one query vertex at a time over *every* unused data vertex
    (no adjacency lists, no intersections); each condition of the definition is
    tested as soon as all of its vertices are assigned.  Returns the sorted
    (M, k) array of tuples indexed by query vertex id.
    """
    n, k = graph.n, query.k
    A = np.zeros((n, n), dtype=bool)
    if graph.m:
        A[graph.edges[:, 0], graph.edges[:, 1]] = True
        A[graph.edges[:, 1], graph.edges[:, 0]] = True
    lab = np.zeros(n, dtype=np.int64) if graph.labels is None else graph.labels.astype(np.int64)
    cons = list(constraints)
    maps = np.zeros((1, 0), dtype=np.int64)
    for u in range(k):
        rows = np.repeat(maps, n, axis=0)
        col = np.tile(np.arange(n, dtype=np.int64), maps.shape[0])
        ok = np.ones(col.shape[0], dtype=bool)
        for j in range(u):                      # injective
            ok &= rows[:, j] != col
        if query.labels is not None:            # labels
            ok &= lab[col] == int(query.labels[u])
        for a, b in query.edges:                # edges with both ends assigned
            if max(a, b) == u:
                other = min(a, b)
                ok &= A[rows[:, other], col]
        for a, b in cons:                       # f(a) < f(b)
            if max(a, b) == u:
                fa = col if a == u else rows[:, a]
                fb = col if b == u else rows[:, b]
                ok &= fa < fb
        maps = np.concatenate([rows[ok], col[ok, None]], axis=1)
    if maps.shape[0] == 0:
        return np.zeros((0, k), dtype=np.int32)
    maps = maps.astype(np.int32)
    return maps[np.lexsort(maps.T[::-1])]


# --------------------------------------------------------------------- O3
def vf2_count(graph, query) -> int:
    """Number of monomorphisms (edge-preserving injective maps) by networkx VF2."""
    import networkx as nx
    from networkx.algorithms import isomorphism as iso

    G = nx.Graph()
    G.add_nodes_from(range(graph.n))
    G.add_edges_from((int(a), int(b)) for a, b in graph.edges)
    Q = nx.Graph()
    Q.add_nodes_from(range(query.k))
    Q.add_edges_from(query.edges)
    nm = None
    if query.labels is not None:
        lab = np.zeros(graph.n, dtype=np.int64) if graph.labels is None else graph.labels
        for v in range(graph.n):
            G.nodes[v]["l"] = int(lab[v])
        for u in range(query.k):
            Q.nodes[u]["l"] = int(query.labels[u])
        nm = iso.categorical_node_match("l", -1)
    gm = iso.GraphMatcher(G, Q, node_match=nm)
    return sum(1 for _ in gm.subgraph_monomorphisms_iter())
