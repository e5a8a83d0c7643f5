"""Seeded synthetic inputs shared by the oracle tests, the CUDA-path tests and bench.py.

This module holds none of the matching method's arithmetic: it only draws edge
lists (as simple undirected graphs: canonical u < v pairs, no self-loops, no
duplicates, sorted) and names query patterns.  The paper's data graphs (Table I,
PAPER.md:414-430) and query patterns (Fig. 8, lost in extraction)
are not available; the recipes below are the synthetic stand-ins fixed in
SURVEY.md Appendix A.2 / section 8(d) and restated in DESIGN.md.

Every generator is a pure function of its arguments (seed included).  The heavy
samplers live in ``gen.c`` (splitmix64 counter-based draws, so the result does
not depend on the thread count).
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from dataclasses import dataclass
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libtdfsgen.so")
_lib = None


def build_gen(force: bool = False) -> str:
    """Compile gen.c into libtdfsgen.so (plain gcc, -O2, pthreads)."""
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-pthread", "-o", tmp, src, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def _gen():
    global _lib
    if _lib is None:
        build_gen()
        lib = ctypes.CDLL(_SO)
        u64p = ctypes.POINTER(ctypes.c_uint64)
        lib.tdfs_gen_rmat.restype = ctypes.c_int64
        lib.tdfs_gen_rmat.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_double, ctypes.c_double,
                                      ctypes.c_double, ctypes.c_uint64, ctypes.c_int, u64p]
        lib.tdfs_gen_chung_lu.restype = ctypes.c_int64
        lib.tdfs_gen_chung_lu.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_double, ctypes.c_double,
                                          ctypes.c_double, ctypes.c_uint64, ctypes.c_int, u64p]
        lib.tdfs_chung_lu_weight_sum.restype = ctypes.c_double
        lib.tdfs_chung_lu_weight_sum.argtypes = [ctypes.c_int64, ctypes.c_double, ctypes.c_double, ctypes.c_double]
        lib.tdfs_gen_finish.restype = ctypes.c_int64
        lib.tdfs_gen_finish.argtypes = [u64p, ctypes.c_int64]
        lib.tdfs_gen_labels.restype = None
        lib.tdfs_gen_labels.argtypes = [ctypes.c_int64, ctypes.c_int, ctypes.c_uint64,
                                        ctypes.POINTER(ctypes.c_uint8)]
        _lib = lib
    return _lib


def _threads() -> int:
    return max(1, min(64, os.cpu_count() or 1))


@dataclass
class Graph:
    """A simple undirected graph: ``edges`` is an (m, 2) int32 array of sorted, unique u < v pairs."""
    n: int
    edges: np.ndarray
    labels: Optional[np.ndarray] = None  # uint8[n] or None (unlabeled)
    name: str = ""

    @property
    def m(self) -> int:
        return int(self.edges.shape[0])

    def with_labels(self, num_labels: int, seed: int) -> "Graph":
        return Graph(self.n, self.edges, random_labels(self.n, num_labels, seed),
                     f"{self.name}+L{num_labels}")


def _from_keys(keys: np.ndarray, n: int, name: str) -> Graph:
    e = np.empty((keys.shape[0], 2), dtype=np.int32)
    e[:, 0] = (keys >> np.uint64(32)).astype(np.int32)
    e[:, 1] = (keys & np.uint64(0xFFFFFFFF)).astype(np.int32)
    return Graph(n, e, None, name)


def from_edge_list(n: int, pairs: Sequence[Tuple[int, int]], name: str = "custom",
                   labels: Optional[Sequence[int]] = None) -> Graph:
    """Simple-graph canonicalisation of a small explicit edge list."""
    s = set()
    for a, b in pairs:
        a, b = int(a), int(b)
        if a == b:
            continue
        s.add((min(a, b), max(a, b)))
    e = np.array(sorted(s), dtype=np.int32).reshape(-1, 2)
    lab = None if labels is None else np.asarray(labels, dtype=np.uint8)
    return Graph(n, e, lab, name)


def to_csr(g: Graph):
    """Input-format conversion (symmetric CSR of a simple graph): offs int64[n+1], adj int32[2m]."""
    a = np.concatenate([g.edges[:, 0], g.edges[:, 1]]).astype(np.int64)
    b = np.concatenate([g.edges[:, 1], g.edges[:, 0]]).astype(np.int64)
    idx = np.lexsort((b, a))
    cnt = np.bincount(a, minlength=g.n)
    offs = np.zeros(g.n + 1, np.int64)
    np.cumsum(cnt, out=offs[1:])
    return offs, np.ascontiguousarray(b[idx].astype(np.int32))


def random_labels(n: int, num_labels: int, seed: int) -> np.ndarray:
    out = np.empty(n, dtype=np.uint8)
    _gen().tdfs_gen_labels(n, int(num_labels), int(seed), out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)))
    return out


# ------------------------------------------------------------------ families
def erdos_renyi(n: int, m: int, seed: int) -> Graph:
    """G(n, m): the first m distinct pairs of a seeded stream of uniform pairs."""
    rng = np.random.default_rng(seed)
    keys: List[np.ndarray] = []
    have = 0
    order_keys = np.empty(0, dtype=np.uint64)
    max_m = n * (n - 1) // 2
    if m > max_m:
        raise ValueError("m too large")
    while have < m:
        k = max(1024, 2 * (m - have))
        a = rng.integers(0, n, size=k, dtype=np.int64)
        b = rng.integers(0, n, size=k, dtype=np.int64)
        ok = a != b
        lo = np.minimum(a, b)[ok].astype(np.uint64)
        hi = np.maximum(a, b)[ok].astype(np.uint64)
        order_keys = np.concatenate([order_keys, (lo << np.uint64(32)) | hi])
        _, first = np.unique(order_keys, return_index=True)
        have = first.shape[0]
    _, first = np.unique(order_keys, return_index=True)
    chosen = np.sort(order_keys[np.sort(first)[:m]])
    return _from_keys(chosen, n, f"er_n{n}_m{m}_s{seed}")


def rmat(scale: int, edge_factor: float, seed: int, a: float = 0.57, b: float = 0.19, c: float = 0.19) -> Graph:
    """Graph500-style R-MAT: edge_factor * 2^scale samples, ids permuted, simple graph."""
    n = 1 << scale
    ns = int(round(edge_factor * n))
    keys = np.empty(ns, dtype=np.uint64)
    cnt = _gen().tdfs_gen_rmat(scale, ns, a, b, c, int(seed), _threads(),
                               keys.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)))
    if cnt < 0:
        raise MemoryError("rmat")
    return _from_keys(keys[:cnt].copy(), n, f"rmat_s{scale}_ef{edge_factor:g}_s{seed}")


def chung_lu(n: int, m_target: int, gamma: float, wmax: float, seed: int, oversample: float = 1.04) -> Graph:
    """Chung-Lu power law: w_i = wmax ((i+i0)/i0)^(-1/(gamma-1)), i0 solved so sum(w) = 2 m_target."""
    lib = _gen()
    target = 2.0 * m_target
    lo, hi = 1e-3, float(n)
    for _ in range(48):  # sum is increasing in i0
        mid = math.sqrt(lo * hi)
        if lib.tdfs_chung_lu_weight_sum(n, gamma, wmax, mid) < target:
            lo = mid
        else:
            hi = mid
    i0 = math.sqrt(lo * hi)
    ns = int(round(oversample * m_target))
    keys = np.empty(ns, dtype=np.uint64)
    cnt = lib.tdfs_gen_chung_lu(n, ns, gamma, wmax, i0, int(seed), _threads(),
                                keys.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)))
    if cnt < 0:
        raise MemoryError("chung_lu")
    g = _from_keys(keys[:cnt].copy(), n, f"cl_n{n}_g{gamma:g}_s{seed}")
    return g


def complete(n: int) -> Graph:
    return from_edge_list(n, [(i, j) for i in range(n) for j in range(i + 1, n)], f"K{n}")


def complete_bipartite(a: int, b: int) -> Graph:
    return from_edge_list(a + b, [(i, a + j) for i in range(a) for j in range(b)], f"K{a},{b}")


def grid(r: int, c: int) -> Graph:
    pairs = []
    for i in range(r):
        for j in range(c):
            v = i * c + j
            if j + 1 < c:
                pairs.append((v, v + 1))
            if i + 1 < r:
                pairs.append((v, v + c))
    return from_edge_list(r * c, pairs, f"grid{r}x{c}")


def small_random(n: int, p: float, seed: int) -> Graph:
    rng = np.random.default_rng(seed)
    pairs = [(i, j) for i in range(n) for j in range(i + 1, n) if rng.random() < p]
    return from_edge_list(n, pairs, f"gnp{n}_{p:g}_s{seed}")


# Fig. 1 of the paper, reconstructed in SURVEY.md App. A.1.
# Data vertices v1..v7 are ids 0..6 (v_i -> i-1).
FIG1_DATA_EDGES = [(1, 2), (1, 3), (1, 4), (2, 3), (2, 4), (3, 4), (2, 7), (3, 7), (4, 5), (5, 6)]


def fig1_data() -> Graph:
    return from_edge_list(7, [(a - 1, b - 1) for a, b in FIG1_DATA_EDGES], "fig1")


def plant(g: Graph, pattern: Graph, seed: int) -> Graph:
    """Copy `pattern` onto distinct random vertices of `g` (adds its edges)."""
    rng = np.random.default_rng(seed)
    where = rng.choice(g.n, size=pattern.n, replace=False)
    extra = where[pattern.edges.astype(np.int64)]
    lo = np.minimum(extra[:, 0], extra[:, 1]).astype(np.uint64)
    hi = np.maximum(extra[:, 0], extra[:, 1]).astype(np.uint64)
    keys = np.concatenate([(g.edges[:, 0].astype(np.uint64) << np.uint64(32)) | g.edges[:, 1].astype(np.uint64),
                           (lo << np.uint64(32)) | hi])
    keys = np.unique(keys)
    out = _from_keys(keys, g.n, f"{g.name}+plant({pattern.name})")
    out.labels = g.labels
    return out


# ------------------------------------------------------------------- queries
@dataclass
class Query:
    name: str
    k: int
    edges: List[Tuple[int, int]]
    labels: Optional[List[int]] = None

    def with_labels(self, labels: Sequence[int]) -> "Query":
        return Query(self.name + "_lab", self.k, list(self.edges), list(int(x) for x in labels))


def _clique(k):
    return [(i, j) for i in range(k) for j in range(i + 1, k)]


def _cycle(k):
    return [(i, (i + 1) % k) for i in range(k)]


def _wheel(rim):
    return [(0, i) for i in range(1, rim + 1)] + [(i, i % rim + 1) for i in range(1, rim + 1)]


QUERIES: Dict[str, Query] = {}


def _q(name, k, edges):
    QUERIES[name] = Query(name, k, [tuple(e) for e in edges])


_q("edge", 2, [(0, 1)])
_q("wedge", 3, [(0, 1), (0, 2)])
_q("triangle", 3, _clique(3))
_q("path3", 4, [(0, 1), (1, 2), (2, 3)])
_q("star3", 4, [(0, 1), (0, 2), (0, 3)])
_q("c4", 4, _cycle(4))
_q("diamond", 4, [(0, 1), (0, 2), (1, 2), (1, 3), (2, 3)])
_q("tailed_triangle", 4, [(0, 1), (0, 2), (1, 2), (2, 3)])
_q("k4", 4, _clique(4))
_q("house", 5, [(0, 1), (1, 2), (2, 3), (3, 0), (0, 4), (1, 4)])
_q("c5", 5, _cycle(5))
_q("k5", 5, _clique(5))
_q("star4", 5, [(0, 1), (0, 2), (0, 3), (0, 4)])
# Fig. 1 query: u1..u5 -> 0..4
_q("fig1_q", 5, [(0, 1), (0, 2), (1, 2), (0, 3), (2, 3), (1, 4), (3, 4)])
_q("prism", 6, [(0, 1), (1, 2), (0, 2), (3, 4), (4, 5), (3, 5), (0, 3), (1, 4), (2, 5)])
_q("w5", 6, _wheel(5))
_q("c6", 6, _cycle(6))
_q("k6", 6, _clique(6))
_q("k6_minus_e", 6, [e for e in _clique(6) if e != (4, 5)])
_q("w6", 7, _wheel(6))
_q("two_k4", 7, _clique(4) + [(3, 4), (3, 5), (3, 6), (4, 5), (4, 6), (5, 6)])
_q("k7", 7, _clique(7))
_q("k7_minus_e", 7, [e for e in _clique(7) if e != (5, 6)])
_q("k8", 8, _clique(8))
_q("k8_minus_e", 8, [e for e in _clique(8) if e != (6, 7)])
_q("c8", 8, _cycle(8))


def query(name: str) -> Query:
    return QUERIES[name]


def labeled_query(name: str, num_labels: int) -> Query:
    """Label rule of PAPER.md:444 adapted per DESIGN.md: label(u_i) = i mod num_labels (0-based i)."""
    q = QUERIES[name]
    return q.with_labels([i % num_labels for i in range(q.k)])


# -------------------------------------------------- the BASELINE.json configs
def config_graph(cfg: int, **over) -> Graph:
    """The synthetic data graph of BASELINE.json configs[cfg-1] (recipes in DESIGN.md)."""
    if cfg == 1:
        return erdos_renyi(over.get("n", 2000), over.get("m", 10000), over.get("seed", 1))
    if cfg == 2:
        return rmat(18, 16, over.get("seed", 1))
    if cfg == 3:
        return rmat(20, 6, over.get("seed", 1))
    if cfg == 4:
        g = chung_lu(4_000_000, 34_700_000, 2.2, 15000.0, over.get("seed", 7))
        return g.with_labels(8, over.get("label_seed", 11))
    if cfg == 5:
        return rmat(22, over.get("edge_factor", 30), over.get("seed", 1))
    raise ValueError(cfg)


# Query sets bench.py times per config.  BASELINE.json names larger sets for configs 3-5; their full
# counts take 16 min (C3 house / c5) to days (C4 w6 / two_k4 ~1.3 h, C5 k5 ~3.3 h, k6 ~11 days) on one
# B200 (sampled-roots estimates, profiles/configs_probe_r02.txt), so the bench lines are gated to the
# queries whose full time-to-count is seconds to minutes (SURVEY.md 8(d) gating rule).
BENCH_QUERIES = {
    1: ["fig1_q"],
    2: ["triangle", "c4", "diamond", "tailed_triangle", "k4"],
    3: ["k5"],
    4: ["prism", "w5"],
    5: ["k4"],
}

CONFIG_QUERIES = {
    1: ["fig1_q"],
    2: ["triangle", "c4", "diamond", "tailed_triangle", "k4"],
    3: ["house", "c5", "k5"],
    4: ["prism", "w5", "w6", "two_k4"],
    5: ["k6", "k7", "k8", "k6_minus_e", "k7_minus_e", "k8_minus_e"],
}
