/*
 * oracle/oracle.cpp -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU subgraph matcher used to check the CUDA
 * path.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  It shares no code, header, table or
 * helper with paper_conf_icde_yuan0ha0024_b200/ (the product), and never
 * reads anything the product computes.
 *
 * What it computes (the plain definition):
 *   M(G,Q,C) = { f : V_Q -> V  |  f injective;
 *                                 for all (u,u') in E_Q: {f(u), f(u')} in E;
 *                                 for all u: L(f(u)) = L_Q(u)   (when Q is labeled);
 *                                 for all (a,b) in C: f(a) < f(b) }
 * following PAPER.md:54-73 (Section II, Algorithm 1), Eq. (1) at PAPER.md:77-79,
 * the injectivity note and label-filtered N(v) at PAPER.md:82, and the
 * symmetry-breaking id(u_i) < id(u_j) constraints of PAPER.md:29 / :460.
 *
 * Algorithm 1 is written out literally: a matching order pi, then a recursive
 * enumerate(S, i) whose candidate set is Eq. (1), the intersection over the
 * backward neighbours B^pi(u_i) of their adjacency lists (std::set_intersection,
 * a library primitive), followed by the injectivity, label and constraint
 * checks of the definition.  When B^pi(u_i) is empty the intersection over the
 * empty family is V.
 *
 * Extras used only for parity of the CUDA path's statistics (never for M):
 *  - an optional degree filter deg(v) >= deg_Q(u) (sound),
 *    placed as in DESIGN.md reading R8 (positions 0 and 1 always, later
 *    positions only when deg_Q(u) > |B^pi(u)|);
 *  - per-position node counts and the algorithmic byte count W of
 *    SURVEY.md 8(d) (sum over internal prefixes of 4*|operand| + 16 bytes), and the
 *    roofline bytes of DESIGN.md R32 (smallest Eq. (1) source per extension);
 *  - a restriction of the root edge (f(pi_0), f(pi_1)) to those whose rank in
 *    the lexicographic order of directed edges is = r (mod W_shard), used for
 *    sampled parity and the shard-sum invariant.
 *
 * Automorphisms (PAPER.md:29, :460 use BLISS) are computed here by brute force
 * over all k! permutations (k <= 8), and the symmetry-breaking constraint set
 * is built by the stabilizer chain of DESIGN.md reading R3.
 */
#include <algorithm>
#include <atomic>
#include <cstdint>
#include <climits>
#include <cstring>
#include <mutex>
#include <thread>
#include <vector>

namespace {

struct DataGraph {
  int64_t n = 0;
  std::vector<std::vector<int32_t>> adj;  // sorted neighbour lists N(v)
  std::vector<int64_t> edge_rank0;        // number of directed edges (a,b) with a < v
  const uint8_t* label = nullptr;         // NULL: unlabeled (every L(v) = 0)
};

struct QueryGraph {
  int k = 0;
  std::vector<std::vector<int>> nbr;  // query adjacency
  std::vector<int> label;             // -1 when Q is unlabeled (no label test)
  std::vector<std::pair<int, int>> constraints;  // f(a) < f(b)
};

struct Job {
  const DataGraph* g;
  const QueryGraph* q;
  std::vector<int> order;               // pi: position -> query vertex
  std::vector<std::vector<int>> bwd;    // B^pi(u_i) as positions
  /* constraints checked at position i: (j, +1) means f(pi_j) < v, (j, -1) means v < f(pi_j) */
  std::vector<std::vector<std::pair<int, int>>> cons_at;
  bool deg_filter;
  int shard_rank, shard_world;
  int64_t max_out;                      // tuple capacity (0: count only)
  int32_t* out;                         // tuples indexed by query vertex id
};

struct Acc {
  uint64_t count = 0;
  uint64_t nodes[9] = {0};
  uint64_t wbytes = 0;
  uint64_t sbytes = 0;   /* R32 roofline bytes */
  std::vector<int32_t> tuples;  // local tuples (enumerate)
  std::vector<const std::vector<int32_t>*> raw;  // per position: Eq. (1) result before the checks
};

int64_t degree(const DataGraph& g, int32_t v) { return (int64_t)g.adj[v].size(); }

int query_degree(const QueryGraph& q, int u) { return (int)q.nbr[u].size(); }

int degree_threshold(const Job& J, int i);

/* Degree filter placement, reading R8. */
bool degree_ok(const Job& J, int i, int32_t v) {
  if (!J.deg_filter) return true;
  int u = J.order[i];
  int dq = query_degree(*J.q, u);
  bool applies = (i <= 1) || (dq > (int)J.bwd[i].size());
  return !applies || degree(*J.g, v) >= dq;
}

/* The checks of the definition for appending v as f(pi_i) to S. */
bool admissible(const Job& J, const std::vector<int32_t>& S, int i, int32_t v) {
  const QueryGraph& q = *J.q;
  int u = J.order[i];
  for (int j = 0; j < i; j++)                  /* injectivity */
    if (S[j] == v) return false;
  if (q.label[u] >= 0) {                       /* label */
    int lv = J.g->label ? (int)J.g->label[v] : 0;
    if (lv != q.label[u]) return false;
  }
  for (auto& c : J.cons_at[i]) {               /* f(a) < f(b) */
    if (c.second > 0 && !(S[c.first] < v)) return false;
    if (c.second < 0 && !(v < S[c.first])) return false;
  }
  return degree_ok(J, i, v);
}

/* Eq. (1): C_S(u_i) = intersection of N(S[u_j]) over u_j in B^pi(u_i).
 * Returns a pointer to the candidate list (N(S[u_j]) itself when |B| = 1). */
const std::vector<int32_t>* candidates(const Job& J, const std::vector<int32_t>& S, int i,
                                       std::vector<int32_t>& C) {
  const DataGraph& g = *J.g;
  C.clear();
  if (J.bwd[i].empty()) {                      /* empty family: all of V */
    for (int64_t v = 0; v < g.n; v++) C.push_back((int32_t)v);
    return &C;
  }
  if (J.bwd[i].size() == 1) return &g.adj[S[J.bwd[i][0]]];
  C = g.adj[S[J.bwd[i][0]]];
  std::vector<int32_t> tmp;
  for (size_t t = 1; t < J.bwd[i].size(); t++) {
    const auto& L = g.adj[S[J.bwd[i][t]]];
    tmp.clear();
    std::set_intersection(C.begin(), C.end(), L.begin(), L.end(), std::back_inserter(tmp));
    C.swap(tmp);
  }
  return &C;
}

bool in_shard(const Job& J, int32_t v0, int32_t v1) {
  if (J.shard_world <= 1) return true;
  const auto& L = J.g->adj[v0];
  int64_t pos = std::lower_bound(L.begin(), L.end(), v1) - L.begin();
  int64_t rank = J.g->edge_rank0[v0] + pos;  /* lexicographic rank of (v0,v1) */
  return rank % J.shard_world == J.shard_rank;
}

/* Is the degree filter applied at position i (R8), and with which threshold (0 = none)? */
int degree_threshold(const Job& J, int i) {
  if (!J.deg_filter) return 0;
  int dq = query_degree(*J.q, J.order[i]);
  return (i <= 1 || dq > (int)J.bwd[i].size()) ? dq : 0;
}

/* R32: may the candidate set C(r) of an earlier position r -- the ids that passed
 * every check at r -- serve as an Eq. (1) source for position i ("if
 * B(u_j) is a subset of B(u_i) ... C(u_i) can be computed from C(u_j)")?  Only if every check
 * made at r also holds for each candidate of i, so that C(r) contains C(i):
 *   adjacency: B(r) is a subset of B(i);
 *   label:     r has no label test, or i tests the same label;
 *   degree:    r's threshold is at most i's own, or at most |B(i)| (a candidate of i is adjacent
 *              to |B(i)| distinct matched vertices);
 *   constraints: every window bound (j, sign) checked at r is also checked at i;
 *   injectivity: checked at i against every earlier position anyway. */
bool source_ok(const Job& J, int r, int i) {
  for (int pj : J.bwd[r])
    if (std::find(J.bwd[i].begin(), J.bwd[i].end(), pj) == J.bwd[i].end()) return false;
  const int lr = J.q->label[J.order[r]], li = J.q->label[J.order[i]];
  if (lr >= 0 && lr != li) return false;
  const int dr = degree_threshold(J, r), di = degree_threshold(J, i);
  if (dr > std::max(di, (int)J.bwd[i].size())) return false;
  for (auto& c : J.cons_at[r])
    if (std::find(J.cons_at[i].begin(), J.cons_at[i].end(), c) == J.cons_at[i].end()) return false;
  return true;
}

/* Algorithm 1, procedure enumerate(S, i, pi, G_Q, G). */
void enumerate(const Job& J, std::vector<int32_t>& S, int i, Acc& acc,
               std::vector<std::vector<int32_t>>& cbuf) {
  const int k = J.q->k;
  const std::vector<int32_t>& C = *candidates(J, S, i, cbuf[i]);  /* line 3 */
  acc.raw[i] = &C;
  if (i >= 2) {                                        /* W of SURVEY 8(d) */
    for (int pj : J.bwd[i]) acc.wbytes += 4ull * (uint64_t)degree(*J.g, S[pj]) + 16ull;
    /* R32 roofline bytes: 16 B per backward operand + 4 B x the smallest SOURCE of Eq. (1)
     * restricted to the ids the constraints already allow (lo <= w < hi).  Sources: every
     * backward operand N(S[j]), and the candidate set C(r) of every stored earlier position
     * r (2 <= r <= k-2) allowed by source_ok (set-intersection reuse).
     * No id bytes for a count-only last position: one source that alone is C(i) up to the
     * matched vertices (a single operand, or a C(r) with B(r) = B(i)) and no label or degree
     * test left at i. */
    int64_t lo = 0, hi = (int64_t)INT32_MAX + 1;
    for (auto& c : J.cons_at[i]) {
      if (c.second > 0) lo = std::max<int64_t>(lo, (int64_t)S[c.first] + 1);
      else hi = std::min<int64_t>(hi, (int64_t)S[c.first]);
    }
    uint64_t mn = UINT64_MAX;
    for (int pj : J.bwd[i]) {
      const auto& L = J.g->adj[S[pj]];
      uint64_t len = 0;
      if (lo < hi) len = (uint64_t)(std::lower_bound(L.begin(), L.end(), hi) - std::lower_bound(L.begin(), L.end(), lo));
      mn = std::min(mn, len);
    }
    const int li = J.q->label[J.order[i]];
    const bool no_test = li < 0 && degree_threshold(J, i) == 0;
    bool count_only = (i + 1 == k) && J.bwd[i].size() == 1 && no_test;
    for (int r = 2; r < i && r <= k - 2; r++) {
      if (!source_ok(J, r, i)) continue;
      uint64_t len = 0;  /* |C(r) within [lo, hi)|: ids of the raw list that passed r's checks */
      for (int32_t v : *acc.raw[r])
        if (v >= lo && v < hi && admissible(J, S, r, v)) len++;
      mn = std::min(mn, len);
      const bool same_b = J.bwd[r].size() == J.bwd[i].size();
      const int lr = J.q->label[J.order[r]];
      const bool label_done = li < 0 || lr == li;
      const int di = degree_threshold(J, i);
      if (i + 1 == k && same_b && label_done && (di == 0 || degree_threshold(J, r) >= di)) count_only = true;
    }
    acc.sbytes += 16ull * J.bwd[i].size() + ((count_only || lo >= hi || mn == UINT64_MAX) ? 0ull : 4ull * mn);
  }
  for (size_t t = 0; t < C.size(); t++) {              /* line 4 */
    int32_t v = C[t];
    if (!admissible(J, S, i, v)) continue;
    if (i == 1 && !in_shard(J, S[0], v)) continue;
    S[i] = v;                                          /* line 5 */
    acc.nodes[i]++;
    if (i + 1 == k) {                                  /* line 6: output S */
      acc.count++;
      if (J.max_out > 0) {
        for (int j = 0; j < k; j++) acc.tuples.push_back(0);
        size_t base = acc.tuples.size() - k;
        for (int j = 0; j < k; j++) acc.tuples[base + J.order[j]] = S[j];
      }
    } else {
      enumerate(J, S, i + 1, acc, cbuf);               /* line 7 */
    }
  }                                                    /* line 8: pop */
}

/* Oracle's own matching order: BFS from the highest-degree query
 * vertex, neighbours visited in increasing id.  Deliberately not
 * the product planner's greedy order. */
std::vector<int> bfs_order(const QueryGraph& q) {
  std::vector<int> order;
  std::vector<char> seen(q.k, 0);
  while ((int)order.size() < q.k) {
    int start = -1;
    for (int u = 0; u < q.k; u++)
      if (!seen[u] && (start < 0 || q.nbr[u].size() > q.nbr[start].size())) start = u;
    std::vector<int> fifo{start};
    seen[start] = 1;
    for (size_t h = 0; h < fifo.size(); h++) {
      int u = fifo[h];
      order.push_back(u);
      std::vector<int> ns = q.nbr[u];
      std::sort(ns.begin(), ns.end());
      for (int w : ns)
        if (!seen[w]) { seen[w] = 1; fifo.push_back(w); }
    }
  }
  return order;
}

bool build_query(int k, int nqe, const int32_t* qedges, const int32_t* qlabels, int nc,
                 const int32_t* cons, QueryGraph& q) {
  if (k < 1 || k > 8) return false;
  q.k = k;
  q.nbr.assign(k, {});
  for (int e = 0; e < nqe; e++) {
    int a = qedges[2 * e], b = qedges[2 * e + 1];
    if (a < 0 || b < 0 || a >= k || b >= k || a == b) return false;
    if (std::find(q.nbr[a].begin(), q.nbr[a].end(), b) != q.nbr[a].end()) continue;
    q.nbr[a].push_back(b);
    q.nbr[b].push_back(a);
  }
  q.label.assign(k, -1);
  if (qlabels)
    for (int u = 0; u < k; u++) q.label[u] = qlabels[u];
  for (int c = 0; c < nc; c++) {
    int a = cons[2 * c], b = cons[2 * c + 1];
    if (a < 0 || b < 0 || a >= k || b >= k || a == b) return false;
    q.constraints.push_back({a, b});
  }
  return true;
}

void build_data(int64_t n, int64_t m, const int32_t* eu, const int32_t* ev, const uint8_t* label,
                DataGraph& g) {
  g.n = n;
  g.adj.assign(n, {});
  for (int64_t e = 0; e < m; e++) {
    int32_t a = eu[e], b = ev[e];
    if (a == b) continue;
    g.adj[a].push_back(b);
    g.adj[b].push_back(a);
  }
  g.edge_rank0.assign(n + 1, 0);
  for (int64_t v = 0; v < n; v++) {
    auto& L = g.adj[v];
    std::sort(L.begin(), L.end());
    L.erase(std::unique(L.begin(), L.end()), L.end());
    g.edge_rank0[v + 1] = g.edge_rank0[v] + (int64_t)L.size();
  }
  g.label = label;
}

}  // namespace

extern "C" {

/*
 * Count (and optionally enumerate) M(G, Q, C).
 *  edges: m undirected pairs (eu[i], ev[i]); duplicates / both directions are
 *         fine (N(v) is the set of neighbours).
 *  order: NULL = oracle BFS order; else a permutation of 0..k-1.
 *  out_nodes[i] (i < k): number of admissible prefixes of length i+1.
 *  out_w: algorithmic adjacency bytes W.
 *  roots [root_lo, root_hi): only f(pi_0) in this range (root_hi < 0: all).
 * Returns 0 on success, -1 on bad arguments, 1 if more than max_out tuples
 * exist (count still exact; first max_out tuples in DFS order written).
 */
static int match_on(const DataGraph& g,
                 int k, int nqe, const int32_t* qedges, const int32_t* qlabels,
                 int nc, const int32_t* cons, const int32_t* order, int deg_filter,
                 int shard_rank, int shard_world, int64_t root_lo, int64_t root_hi,
                 int nthreads, int64_t max_out, int32_t* out_tuples,
                 uint64_t* out_count, uint64_t* out_nodes, uint64_t* out_w, uint64_t* out_stream) {
  QueryGraph q;
  if (!build_query(k, nqe, qedges, qlabels, nc, cons, q)) return -1;
  if (shard_world < 1 || shard_rank < 0 || shard_rank >= shard_world) return -1;
  const int64_t n = g.n;
  Job J;
  J.g = &g;
  J.q = &q;
  if (order) {
    std::vector<char> seen(k, 0);
    for (int i = 0; i < k; i++) {
      if (order[i] < 0 || order[i] >= k || seen[order[i]]) return -1;
      seen[order[i]] = 1;
      J.order.push_back(order[i]);
    }
  } else {
    J.order = bfs_order(q);
  }
  std::vector<int> pos(k);
  for (int i = 0; i < k; i++) pos[J.order[i]] = i;
  J.bwd.assign(k, {});
  for (int i = 0; i < k; i++)        /* B^pi(u_i) = { u_j : j < i, (u_j,u_i) in E_Q } */
    for (int w : q.nbr[J.order[i]])
      if (pos[w] < i) J.bwd[i].push_back(pos[w]);
  for (int i = 0; i < k; i++) std::sort(J.bwd[i].begin(), J.bwd[i].end());
  /* each constraint (a,b) is checked where its later endpoint is matched */
  J.cons_at.assign(k, {});
  for (auto& c : q.constraints) {
    int pa = pos[c.first], pb = pos[c.second];
    if (pa > pb) J.cons_at[pa].push_back({pb, -1});   /* f(a)=v must be < f(b) */
    else J.cons_at[pb].push_back({pa, +1});           /* f(b)=v must be > f(a) */
  }
  J.deg_filter = deg_filter != 0;
  J.shard_rank = shard_rank;
  J.shard_world = shard_world;
  J.max_out = max_out;
  J.out = out_tuples;

  int64_t lo = std::max<int64_t>(0, root_lo), hi = root_hi < 0 ? n : std::min<int64_t>(n, root_hi);
  if (nthreads < 1) nthreads = 1;
  if (max_out > 0) nthreads = 1;  /* enumerate: one thread, deterministic DFS order */

  std::vector<Acc> accs(nthreads);
  std::atomic<int64_t> next(lo);
  auto worker = [&](int t) {
    Acc& acc = accs[t];
    acc.raw.assign(k, nullptr);
    std::vector<int32_t> S(k, -1);
    std::vector<std::vector<int32_t>> cbuf(k);
    std::vector<int32_t> C0;
    for (;;) {
      int64_t r = next.fetch_add(1);
      if (r >= hi) break;
      /* position 0: C_S(u_1) over the empty backward set is V; handle root r */
      int32_t v = (int32_t)r;
      if (!J.bwd[0].empty()) continue;  /* never: pi_0 has no earlier vertex */
      if (!admissible(J, S, 0, v)) continue;
      S[0] = v;
      acc.nodes[0]++;
      if (k == 1) {
        acc.count++;
        if (max_out > 0) acc.tuples.push_back(v);
        continue;
      }
      enumerate(J, S, 1, acc, cbuf);
    }
  };
  if (nthreads == 1) {
    worker(0);
  } else {
    std::vector<std::thread> th;
    for (int t = 0; t < nthreads; t++) th.emplace_back(worker, t);
    for (auto& x : th) x.join();
  }
  uint64_t count = 0, w = 0, sb = 0, nodes[9] = {0};
  for (auto& a : accs) {
    count += a.count;
    w += a.wbytes;
    sb += a.sbytes;
    for (int i = 0; i < 9; i++) nodes[i] += a.nodes[i];
  }
  if (out_count) *out_count = count;
  if (out_w) *out_w = w;
  if (out_stream) *out_stream = sb;
  if (out_nodes)
    for (int i = 0; i < k; i++) out_nodes[i] = nodes[i];
  int rc = 0;
  if (max_out > 0 && out_tuples) {
    const auto& T = accs[0].tuples;
    int64_t have = (int64_t)(T.size() / (size_t)k);
    int64_t wr = std::min<int64_t>(have, max_out);
    std::memcpy(out_tuples, T.data(), sizeof(int32_t) * (size_t)(wr * k));
    if (have > max_out) rc = 1;
  }
  return rc;
}

int oracle_match(int64_t n, int64_t m, const int32_t* eu, const int32_t* ev, const uint8_t* label,
                 int k, int nqe, const int32_t* qedges, const int32_t* qlabels,
                 int nc, const int32_t* cons, const int32_t* order, int deg_filter,
                 int shard_rank, int shard_world, int64_t root_lo, int64_t root_hi,
                 int nthreads, int64_t max_out, int32_t* out_tuples,
                 uint64_t* out_count, uint64_t* out_nodes, uint64_t* out_w, uint64_t* out_stream) {
  DataGraph g;
  build_data(n, m, eu, ev, label, g);
  return match_on(g, k, nqe, qedges, qlabels, nc, cons, order, deg_filter, shard_rank, shard_world, root_lo, root_hi,
                  nthreads, max_out, out_tuples, out_count, out_nodes, out_w, out_stream);
}

/* Build the oracle's adjacency once and run many queries on it (same semantics). */
void* oracle_graph_new(int64_t n, int64_t m, const int32_t* eu, const int32_t* ev, const uint8_t* label) {
  DataGraph* g = new DataGraph;
  build_data(n, m, eu, ev, label, *g);
  return g;
}

void oracle_graph_free(void* g) { delete (DataGraph*)g; }

int oracle_match_g(const void* g, int k, int nqe, const int32_t* qedges, const int32_t* qlabels,
                   int nc, const int32_t* cons, const int32_t* order, int deg_filter,
                   int shard_rank, int shard_world, int64_t root_lo, int64_t root_hi,
                   int nthreads, int64_t max_out, int32_t* out_tuples,
                   uint64_t* out_count, uint64_t* out_nodes, uint64_t* out_w, uint64_t* out_stream) {
  return match_on(*(const DataGraph*)g, k, nqe, qedges, qlabels, nc, cons, order, deg_filter, shard_rank, shard_world,
                  root_lo, root_hi, nthreads, max_out, out_tuples, out_count, out_nodes, out_w, out_stream);
}

/* The oracle's own matching order (for reporting). */
int oracle_order(int k, int nqe, const int32_t* qedges, int32_t* order_out) {
  QueryGraph q;
  if (!build_query(k, nqe, qedges, nullptr, 0, nullptr, q)) return -1;
  auto o = bfs_order(q);
  for (int i = 0; i < k; i++) order_out[i] = o[i];
  return 0;
}

/*
 * Aut(Q) by brute force over all k! permutations (edges and labels preserved),
 * and the stabilizer-chain symmetry-breaking constraints of DESIGN.md R3:
 *   A <- Aut(Q); while |A| > 1: u <- smallest vertex whose A-orbit has > 1
 *   element; add (u, w) for every other w in that orbit; A <- Stab_A(u).
 * Writes |Aut| and up to cap pairs; returns the number of pairs (or -1).
 */
int oracle_automorphisms(int k, int nqe, const int32_t* qedges, const int32_t* qlabels,
                         int64_t* n_aut, int32_t* pairs, int cap) {
  QueryGraph q;
  if (!build_query(k, nqe, qedges, qlabels, 0, nullptr, q)) return -1;
  std::vector<std::vector<char>> A(k, std::vector<char>(k, 0));
  for (int u = 0; u < k; u++)
    for (int w : q.nbr[u]) A[u][w] = 1;
  std::vector<int> p(k);
  for (int i = 0; i < k; i++) p[i] = i;
  std::vector<std::vector<int>> aut;
  do {
    bool ok = true;
    for (int u = 0; u < k && ok; u++) {
      if (q.label[u] != q.label[p[u]]) ok = false;
      for (int w = 0; w < k && ok; w++)
        if (A[u][w] != A[p[u]][p[w]]) ok = false;
    }
    if (ok) aut.push_back(p);
  } while (std::next_permutation(p.begin(), p.end()));
  *n_aut = (int64_t)aut.size();

  int npairs = 0;
  std::vector<std::vector<int>> G = aut;
  while (G.size() > 1) {
    int pick = -1;
    std::vector<int> orbit;
    for (int u = 0; u < k && pick < 0; u++) {
      std::vector<int> o;
      for (auto& s : G) o.push_back(s[u]);
      std::sort(o.begin(), o.end());
      o.erase(std::unique(o.begin(), o.end()), o.end());
      if (o.size() > 1) { pick = u; orbit = o; }
    }
    for (int w : orbit) {
      if (w == pick) continue;
      if (npairs < cap && pairs) { pairs[2 * npairs] = pick; pairs[2 * npairs + 1] = w; }
      npairs++;
    }
    std::vector<std::vector<int>> H;
    for (auto& s : G)
      if (s[pick] == pick) H.push_back(s);
    G.swap(H);
  }
  return npairs;
}

}  // extern "C"
