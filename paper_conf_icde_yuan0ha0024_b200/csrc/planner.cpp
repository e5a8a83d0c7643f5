// Host query planner.
//
//  - matching order pi: start at the query vertex of highest
//    degree, then repeatedly take the unplaced vertex with the most already-placed
//    neighbours (ties: higher degree, then lower id).  Every prefix is connected,
//    so pi_1 is adjacent to pi_0 and the first two positions are matched by the
//    initial edge tasks.
//  - backward neighbours B^pi(u_i) = { u_j : j < i, (u_j, u_i) in E_Q }.
//  - symmetry breaking (the paper uses BLISS): Aut(Q) is found
//    by a depth-first search over label- and adjacency-consistent partial
//    permutations, then the stabilizer chain of DESIGN.md reading R3 turns it into
//    constraints f(a) < f(b).
//  - per-position filters: label, degree
//    only where not implied (R8), constraint windows, injectivity.
#include <algorithm>
#include <cstring>
#include <functional>
#include <string>

#include "internal.h"

struct tdfs_plan {
  tdfs::Plan p;
};

namespace tdfs {
namespace {

struct QueryAdj {
  int k;
  uint8_t a[kMaxK][kMaxK];
  int deg[kMaxK];
  int lab[kMaxK];
};

// All label-preserving automorphisms of the query, by backtracking.
void automorphisms(const QueryAdj& q, std::vector<std::vector<int>>& out) {
  std::vector<int> phi(q.k, -1);
  std::vector<char> used(q.k, 0);
  std::function<void(int)> rec = [&](int u) {
    if (u == q.k) { out.push_back(phi); return; }
    for (int w = 0; w < q.k; w++) {
      if (used[w] || q.deg[w] != q.deg[u] || q.lab[w] != q.lab[u]) continue;
      bool ok = true;
      for (int x = 0; x < u && ok; x++) ok = (q.a[u][x] == q.a[w][phi[x]]);
      if (!ok) continue;
      used[w] = 1; phi[u] = w;
      rec(u + 1);
      used[w] = 0; phi[u] = -1;
    }
  };
  rec(0);
}

// Stabilizer chain (R3): repeatedly fix the smallest vertex with a
// non-trivial orbit and require it to take the smallest id of its orbit.
std::vector<std::pair<int, int>> stabilizer_constraints(int k, std::vector<std::vector<int>> group) {
  std::vector<std::pair<int, int>> cons;
  while (group.size() > 1) {
    int u = -1;
    uint32_t orbit = 0;
    for (int x = 0; x < k && u < 0; x++) {
      uint32_t o = 0;
      for (auto& g : group) o |= 1u << g[x];
      if (__builtin_popcount(o) > 1) { u = x; orbit = o; }
    }
    for (int w = 0; w < k; w++)
      if (w != u && (orbit >> w & 1u)) cons.push_back({u, w});
    std::vector<std::vector<int>> stab;
    for (auto& g : group)
      if (g[u] == u) stab.push_back(g);
    group.swap(stab);
  }
  return cons;
}

std::vector<int> greedy_order(const QueryAdj& q) {
  std::vector<int> order;
  std::vector<char> placed(q.k, 0);
  int first = 0;
  for (int u = 1; u < q.k; u++)
    if (q.deg[u] > q.deg[first]) first = u;
  order.push_back(first);
  placed[first] = 1;
  while ((int)order.size() < q.k) {
    int best = -1, best_b = -1;
    for (int u = 0; u < q.k; u++) {
      if (placed[u]) continue;
      int b = 0;
      for (int w : order) b += q.a[u][w];
      if (b == 0) continue;
      if (b > best_b || (b == best_b && q.deg[u] > q.deg[best])) { best = u; best_b = b; }
    }
    order.push_back(best);
    placed[best] = 1;
  }
  return order;
}

void build_dev(const QueryAdj& q, Plan& P) {
  DevPlan& d = P.dev;
  std::memset(&d, 0, sizeof(d));
  d.k = q.k;
  int pos[kMaxK];
  for (int i = 0; i < q.k; i++) { d.order[i] = P.order[i]; pos[P.order[i]] = i; }
  for (int i = q.k; i < kMaxK; i++) { d.order[i] = -1; d.label[i] = -1; }
  for (int p = 0; p < q.k; p++) {
    int u = P.order[p];
    for (int j = 0; j < p; j++)
      if (q.a[u][P.order[j]]) d.bwd[p] |= 1u << j;
    d.label[p] = P.qlabel.empty() ? -1 : P.qlabel[u];
  }
  d.edge_cons = 0;
  for (auto& c : P.constraints) {  // f(c.first) < f(c.second)
    int pa = pos[c.first], pb = pos[c.second];
    if (pa <= 1 && pb <= 1) {
      int want = (pa == 0) ? +1 : -1;  // +1: S0 < S1
      d.edge_cons = (d.edge_cons == 0 || d.edge_cons == want) ? want : 2;  // 2: contradictory -> empty
    } else if (pb > pa) {
      d.lo_mask[pb] |= 1u << pa;       // v = f(b) must exceed S[pa]
    } else {
      d.hi_mask[pa] |= 1u << pb;       // v = f(a) must be below S[pb]
    }
  }
  for (int p = 0; p < q.k; p++) {
    uint32_t all = (1u << p) - 1u;
    d.inj_mask[p] = all & ~d.bwd[p] & ~d.lo_mask[p] & ~d.hi_mask[p];
    int dq = q.deg[P.order[p]];
    int nb = __builtin_popcount(d.bwd[p]);
    d.deg_min[p] = (p <= 1 || dq > nb) ? dq : 0;
  }
  // Set-intersection result reuse: position p may start from the stored
  // candidate list C(r) of an earlier position r when B(r) is a subset of B(p) -- and, because
  // C(r) is already filtered, when every filter applied at r also holds for p's candidates:
  // same (or no) label, r's degree threshold implied at p, r's constraint window implied at p.
  // Largest B(r) wins (most operands saved), then the latest r.
  for (int p = 0; p < kMaxK; p++) { d.reuse[p] = -1; d.shortcut[p] = 0; }
  for (int p = 3; p < q.k; p++) {
    int best = -1;
    for (int r = 2; r < p && r <= q.k - 2; r++) {
      if ((d.bwd[r] & d.bwd[p]) != d.bwd[r]) continue;
      if (d.label[r] >= 0 && d.label[r] != d.label[p]) continue;
      int nb = __builtin_popcount(d.bwd[p]);
      if (d.deg_min[r] > std::max(d.deg_min[p], nb)) continue;
      if ((d.lo_mask[r] & d.lo_mask[p]) != d.lo_mask[r]) continue;
      if ((d.hi_mask[r] & d.hi_mask[p]) != d.hi_mask[r]) continue;
      d.src_mask[p] |= 1u << r;
      if (best < 0 || __builtin_popcount(d.bwd[r]) >= __builtin_popcount(d.bwd[best])) best = r;
    }
    d.reuse[p] = (int8_t)best;
  }
  // R32 count-only last position (for the roofline bytes, independent of which r is reused)
  if (q.k >= 3) {
    const int p = q.k - 1;
    const bool nolab = d.label[p] < 0, nodeg = d.deg_min[p] == 0;
    bool co = __builtin_popcount(d.bwd[p]) == 1 && nolab && nodeg;
    for (int r = 2; r < p; r++)
      if (((d.src_mask[p] >> r) & 1u) && d.bwd[r] == d.bwd[p] && (nolab || d.label[r] == d.label[p]) &&
          (nodeg || d.deg_min[r] >= d.deg_min[p]))
        co = true;
    d.cnt_only[p] = co;
  }
  // Count-only last position: when one list remains (one backward operand, or a reused C(r)
  // with B(r) = B(p)) and no per-element label/degree test is needed, |C(p)| is the size of
  // the constraint window minus the already-matched vertices inside it (no scan).
  {
    int p = q.k - 1;
    if (p >= 2) {
      int nb = __builtin_popcount(d.bwd[p]);
      bool nolab = d.label[p] < 0, nodeg = d.deg_min[p] == 0;
      if (nb == 1 && nolab && nodeg) d.shortcut[p] |= 2;
      int r = d.reuse[p];
      if (r >= 0 && d.bwd[r] == d.bwd[p] && (nolab || d.label[r] == d.label[p]) &&
          (nodeg || d.deg_min[r] >= d.deg_min[p]))
        d.shortcut[p] |= 1;
    }
  }
  // Leaf staging: the virtual position kVF holds the S[k-2]-independent part of the last
  // position (internal.h).  A superset start C(r) for it follows the reuse rule above with
  // r <= k-2 (all stored lists of the current prefix are alive while level k-2 iterates).
  d.lf_on = 0;
  d.reuse[kVF] = -1;
  d.shortcut[kVF] = 0;
  if (q.k >= 4) {
    const int p = q.k - 1, v = q.k - 2;
    const uint32_t fixm = (1u << v) - 1u;
    d.bwd[kVF] = d.bwd[p] & fixm;
    d.lo_mask[kVF] = d.lo_mask[p] & fixm;
    d.hi_mask[kVF] = d.hi_mask[p] & fixm;
    d.inj_mask[kVF] = d.inj_mask[p] & fixm;
    d.label[kVF] = d.label[p];
    d.deg_min[kVF] = d.deg_min[p];
    d.lf_var = (int8_t)((d.bwd[p] >> v) & 1u);
    d.lf_lo_var = (int8_t)((d.lo_mask[p] >> v) & 1u);
    d.lf_hi_var = (int8_t)((d.hi_mask[p] >> v) & 1u);
    d.lf_inj_var = (int8_t)((d.inj_mask[p] >> v) & 1u);
    d.lf_on = d.bwd[kVF] != 0;
    // F referenced in place: one operand, no per-element filter; injectivity against positions
    // <= k-3 only when the leaf count does not intersect N(S[k-2]) (then it is a subtraction)
    d.lf_byref = (int8_t)(__builtin_popcount(d.bwd[kVF]) == 1 && d.label[kVF] < 0 && d.deg_min[kVF] == 0 &&
                          (d.inj_mask[kVF] == 0 || !d.lf_var));
    int best = -1;
    const int nb = __builtin_popcount(d.bwd[p]);
    for (int r = 2; r <= v; r++) {
      if ((d.bwd[r] & d.bwd[kVF]) != d.bwd[r]) continue;
      if (d.label[r] >= 0 && d.label[r] != d.label[p]) continue;
      if (d.deg_min[r] > std::max(d.deg_min[p], nb)) continue;
      if ((d.lo_mask[r] & d.lo_mask[kVF]) != d.lo_mask[r]) continue;
      if ((d.hi_mask[r] & d.hi_mask[kVF]) != d.hi_mask[r]) continue;
      if (best < 0 || __builtin_popcount(d.bwd[r]) >= __builtin_popcount(d.bwd[best])) best = r;
    }
    d.reuse[kVF] = (int8_t)best;
  }
  d.reuse_enabled = 1;
}

}  // namespace
}  // namespace tdfs

using namespace tdfs;

extern "C" int tdfs_plan_query(int32_t k, int32_t n_qedges, const int32_t* qedges, const int32_t* qlabel,
                               const tdfs_plan_opts* opts, tdfs_plan** out) {
  if (!out) return fail(TDFS_E_INVALID_ARG, "plan: out is NULL");
  if (k < 2 || k > kMaxK) return fail(TDFS_E_QUERY_TOO_LARGE, "plan: k must be in [2, 8]");
  if (n_qedges < 0 || (n_qedges > 0 && !qedges)) return fail(TDFS_E_INVALID_ARG, "plan: bad query edges");
  QueryAdj q;
  std::memset(&q, 0, sizeof(q));
  q.k = k;
  Plan P;
  P.k = k;
  for (int e = 0; e < n_qedges; e++) {
    int a = qedges[2 * e], b = qedges[2 * e + 1];
    if (a < 0 || b < 0 || a >= k || b >= k) return fail(TDFS_E_INVALID_ARG, "plan: query edge endpoint out of range");
    if (a == b) return fail(TDFS_E_INVALID_ARG, "plan: query self-loop");
    if (q.a[a][b]) continue;
    q.a[a][b] = q.a[b][a] = 1;
    q.deg[a]++; q.deg[b]++;
    P.qedges.push_back({std::min(a, b), std::max(a, b)});
  }
  for (int u = 0; u < k; u++) {
    if (qlabel) {
      if (qlabel[u] < 0 || qlabel[u] > 255) return fail(TDFS_E_LABEL_RANGE, "plan: query label outside [0,255]");
      q.lab[u] = qlabel[u];
    } else {
      q.lab[u] = -1;
    }
  }
  if (qlabel) P.qlabel.assign(qlabel, qlabel + k);
  // connectivity
  {
    uint32_t seen = 1u, frontier = 1u;
    while (frontier) {
      uint32_t nxt = 0;
      for (int u = 0; u < k; u++)
        if (frontier >> u & 1u)
          for (int w = 0; w < k; w++)
            if (q.a[u][w] && !(seen >> w & 1u)) nxt |= 1u << w;
      seen |= nxt;
      frontier = nxt;
    }
    if (seen != (1u << k) - 1u) return fail(TDFS_E_QUERY_DISCONNECTED, "plan: query graph is not connected");
  }
  std::vector<std::vector<int>> aut;
  automorphisms(q, aut);
  P.n_aut = (int64_t)aut.size();

  int nc = opts ? opts->n_constraints : -1;
  if (nc < 0) {
    P.constraints = stabilizer_constraints(k, aut);
  } else if (nc > 0) {
    if (!opts->constraints) return fail(TDFS_E_INVALID_ARG, "plan: constraints NULL with n_constraints > 0");
    for (int c = 0; c < nc; c++) {
      int a = opts->constraints[2 * c], b = opts->constraints[2 * c + 1];
      if (a < 0 || b < 0 || a >= k || b >= k || a == b) return fail(TDFS_E_INVALID_ARG, "plan: bad constraint pair");
      P.constraints.push_back({a, b});
    }
  }
  if (opts && opts->order) {
    uint32_t seen = 0;
    for (int i = 0; i < k; i++) {
      int u = opts->order[i];
      if (u < 0 || u >= k || (seen >> u & 1u)) return fail(TDFS_E_INVALID_ARG, "plan: order is not a permutation");
      if (i > 0) {
        bool adj = false;
        for (int j = 0; j < i; j++) adj |= q.a[u][opts->order[j]] != 0;
        if (!adj) return fail(TDFS_E_QUERY_DISCONNECTED, "plan: order prefix is not connected");
      }
      seen |= 1u << u;
      P.order.push_back(u);
    }
  } else {
    P.order = greedy_order(q);
  }
  build_dev(q, P);
  tdfs_plan* h = new (std::nothrow) tdfs_plan;
  if (!h) return fail(TDFS_E_OOM, "plan: host allocation");
  h->p = std::move(P);
  *out = h;
  return TDFS_OK;
}

extern "C" int tdfs_plan_order(const tdfs_plan* p, int32_t* order) {
  if (!p || !order) return fail(TDFS_E_INVALID_ARG, "plan_order: NULL");
  for (int i = 0; i < p->p.k; i++) order[i] = p->p.order[i];
  return TDFS_OK;
}

extern "C" int tdfs_plan_constraints(const tdfs_plan* p, int32_t* pairs, int32_t cap, int32_t* n_out) {
  if (!p || !n_out || cap < 0 || (cap > 0 && !pairs)) return fail(TDFS_E_INVALID_ARG, "plan_constraints: bad args");
  int n = (int)p->p.constraints.size();
  for (int i = 0; i < n && i < cap; i++) {
    pairs[2 * i] = p->p.constraints[i].first;
    pairs[2 * i + 1] = p->p.constraints[i].second;
  }
  *n_out = n;
  return TDFS_OK;
}

extern "C" int tdfs_plan_aut_size(const tdfs_plan* p, int64_t* n_aut) {
  if (!p || !n_aut) return fail(TDFS_E_INVALID_ARG, "plan_aut_size: NULL");
  *n_aut = p->p.n_aut;
  return TDFS_OK;
}

extern "C" int tdfs_plan_k(const tdfs_plan* p, int32_t* k) {
  if (!p || !k) return fail(TDFS_E_INVALID_ARG, "plan_k: NULL");
  *k = p->p.k;
  return TDFS_OK;
}

extern "C" void tdfs_free_plan(tdfs_plan* p) { delete p; }

namespace tdfs {
const Plan* plan_of(const tdfs_plan* p) { return p ? &p->p : nullptr; }
}  // namespace tdfs
