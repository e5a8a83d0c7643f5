// Graph loader: CSR in device memory,
// 32-bit ids, optional labels.  Host-side
// normalisation is multithreaded so that it never dominates a job (the paper's
// point about STMatch's serial host preprocessing).
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <thread>

#include "internal.h"

struct tdfs_graph {
  tdfs::Graph g;
};

namespace tdfs {
namespace {

constexpr int64_t kMaxN = (int64_t)2147483647 - 2;  // -1/-2 are queue sentinels

int cuda_fail(cudaError_t e, const char* what) {
  return fail(TDFS_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

int n_threads() {
  unsigned h = std::thread::hardware_concurrency();
  return (int)std::max(1u, std::min(h, 64u));
}

template <class F>
void parallel_for(int64_t n, F&& f) {
  int T = n_threads();
  if (n < (1 << 16) || T == 1) { f(0, n); return; }
  std::vector<std::thread> th;
  int64_t step = (n + T - 1) / T;
  for (int t = 0; t < T; t++) {
    int64_t lo = t * step, hi = std::min(n, lo + step);
    if (lo >= hi) break;
    th.emplace_back([&f, lo, hi] { f(lo, hi); });
  }
  for (auto& x : th) x.join();
}

// Build a simple symmetric CSR from directed pairs (a[i] -> b[i] and b[i] -> a[i]).
void build_csr(int64_t n, int64_t m, const int32_t* a, const int32_t* b, std::vector<int64_t>& offs,
               std::vector<int32_t>& adj) {
  std::vector<int64_t> deg(n + 1, 0);
  parallel_for(m, [&](int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; i++) {
      if (a[i] == b[i]) continue;
      __atomic_fetch_add(&deg[a[i]], 1, __ATOMIC_RELAXED);
      __atomic_fetch_add(&deg[b[i]], 1, __ATOMIC_RELAXED);
    }
  });
  std::vector<int64_t> start(n + 1, 0);
  for (int64_t v = 0; v < n; v++) start[v + 1] = start[v] + deg[v];
  std::vector<int32_t> tmp((size_t)start[n]);
  std::vector<int64_t> cur(start.begin(), start.end() - 1);
  parallel_for(m, [&](int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; i++) {
      if (a[i] == b[i]) continue;
      tmp[__atomic_fetch_add(&cur[a[i]], 1, __ATOMIC_RELAXED)] = b[i];
      tmp[__atomic_fetch_add(&cur[b[i]], 1, __ATOMIC_RELAXED)] = a[i];
    }
  });
  // sort + dedupe each list in place; new degree into deg[]
  parallel_for(n, [&](int64_t lo, int64_t hi) {
    for (int64_t v = lo; v < hi; v++) {
      int32_t* L = tmp.data() + start[v];
      int64_t d = start[v + 1] - start[v];
      std::sort(L, L + d);
      deg[v] = std::unique(L, L + d) - L;
    }
  });
  offs.assign(n + 1, 0);
  for (int64_t v = 0; v < n; v++) offs[v + 1] = offs[v] + deg[v];
  adj.resize((size_t)offs[n]);
  parallel_for(n, [&](int64_t lo, int64_t hi) {
    for (int64_t v = lo; v < hi; v++)
      std::memcpy(adj.data() + offs[v], tmp.data() + start[v], sizeof(int32_t) * (size_t)deg[v]);
  });
}

// Host validation of a CSR (VALIDATE flag).
int validate_host(int64_t n, int64_t nnz, const int64_t* offs, const int32_t* adj) {
  if (offs[0] != 0 || offs[n] != nnz) return fail(TDFS_E_GRAPH_FORMAT, "validate: offs[0] != 0 or offs[n] != nnz");
  std::atomic<int> bad(0);
  std::atomic<int64_t> where(-1);
  parallel_for(n, [&](int64_t lo, int64_t hi) {
    for (int64_t v = lo; v < hi && !bad.load(std::memory_order_relaxed); v++) {
      if (offs[v + 1] < offs[v]) { bad = 1; where = v; return; }
      for (int64_t e = offs[v]; e < offs[v + 1]; e++) {
        int32_t w = adj[e];
        if (w < 0 || w >= n) { bad = 2; where = v; return; }
        if (w == v) { bad = 3; where = v; return; }
        if (e > offs[v] && adj[e - 1] >= w) { bad = 4; where = v; return; }
        const int32_t* L = adj + offs[w];
        const int32_t* R = adj + offs[w + 1];
        if (offs[w + 1] < offs[w] || !std::binary_search(L, R, (int32_t)v)) { bad = 5; where = v; return; }
      }
    }
  });
  static const char* why[] = {"", "offsets decrease", "id out of range", "self-loop", "list not strictly increasing",
                              "asymmetric edge"};
  if (bad.load()) {
    int code = bad.load() == 2 ? TDFS_E_ID_RANGE : TDFS_E_GRAPH_FORMAT;
    return fail(code, std::string("validate: ") + why[bad.load()] + " at vertex " + std::to_string(where.load()));
  }
  return TDFS_OK;
}

// Cheap host check without VALIDATE: offsets monotone and ids in [0, n) (the kernels index with them).
int check_host_ids(int64_t n, int64_t nnz, const int64_t* offs, const int32_t* adj) {
  if (offs[0] != 0 || offs[n] != nnz) return fail(TDFS_E_GRAPH_FORMAT, "load: offs[0] != 0 or offs[n] != nnz");
  std::atomic<int> bad(0);
  parallel_for(n, [&](int64_t lo, int64_t hi) {
    for (int64_t v = lo; v < hi; v++)
      if (offs[v + 1] < offs[v]) { bad = 1; return; }
  });
  if (bad.load()) return fail(TDFS_E_GRAPH_FORMAT, "load: offsets decrease");
  parallel_for(nnz, [&](int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; i++)
      if (adj[i] < 0 || adj[i] >= n) { bad = 2; return; }
  });
  if (bad.load()) return fail(TDFS_E_ID_RANGE, "load: neighbour id outside [0, n)");
  return TDFS_OK;
}

// ------------------------------------------------------------- device helpers
__global__ void fill_src_kernel(const int64_t* __restrict__ offs, int64_t n, int32_t* __restrict__ src) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t v = warp; v < n; v += nw) {
    int64_t b = offs[v], e = offs[v + 1];
    for (int64_t i = b + lane; i < e; i += 32) src[i] = (int32_t)v;
  }
}

// flags bit0: bad format, bit1: id range; dmax via atomicMax; label max
__global__ void scan_graph_kernel(const int64_t* __restrict__ offs, const int32_t* __restrict__ adj,
                                  const uint8_t* __restrict__ label, int64_t n, int64_t nnz, int validate,
                                  unsigned long long* out /* [0]=dmax [1]=flags [2]=maxlabel */) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  unsigned long long dmax = 0, flags = 0, lmax = 0;
  for (int64_t v = warp; v < n; v += nw) {
    int64_t b = offs[v], e = offs[v + 1];
    if (lane == 0) {
      if (e < b || e > nnz || b < 0) flags |= 1;
      else dmax = max(dmax, (unsigned long long)(e - b));
      if (label) lmax = max(lmax, (unsigned long long)label[v]);
    }
    if (e < b) continue;
    for (int64_t i = b + lane; i < e; i += 32) {
      int32_t w = adj[i];
      if (w < 0 || w >= n) { flags |= 2; continue; }  // always: an id >= n would be read out of bounds
      if (!validate) continue;
      if (w == v || (i > b && adj[i - 1] >= w)) flags |= 1;
      // symmetry: v must be in N(w)
      int64_t lo = offs[w], hi = offs[w + 1];
      while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (adj[mid] < v) lo = mid + 1; else hi = mid;
      }
      if (lo >= offs[w + 1] || adj[lo] != v) flags |= 1;
    }
  }
  if (dmax) atomicMax(&out[0], dmax);
  if (flags) atomicOr(&out[1], flags);
  if (lmax) atomicMax(&out[2], lmax);
}

__global__ void hub_bits_kernel(const int64_t* __restrict__ offs, const int32_t* __restrict__ adj,
                                const int32_t* __restrict__ hub_vertex, long long n_hubs, long long words,
                                uint32_t* __restrict__ bits) {
  for (long long h = blockIdx.x; h < n_hubs; h += gridDim.x) {
    const int32_t v = hub_vertex[h];
    uint32_t* row = bits + h * words;
    for (long long e = offs[v] + threadIdx.x; e < offs[v + 1]; e += blockDim.x) {
      const int32_t w = adj[e];
      atomicOr(row + (w >> 5), 1u << (w & 31));
    }
  }
}

// Hub adjacency bitmaps: the highest-degree vertices (degree >= 256,
// at most `budget` bytes of bitmaps) get an n-bit membership bitmap so that probing
// w in N(hub) during Eq. (1) is one load instead of a binary search over a long list.
int build_hub_bitmaps(Graph& G, cudaStream_t st, const std::vector<int64_t>& offs, int64_t budget) {
  const long long words = (G.n + 31) / 32;
  if (G.n == 0 || words == 0 || budget < 0) return TDFS_OK;
  // default 256 MB -- measured on config 2: 16/64/256/1024 MB -> c4 2029/1416/1350/1350 ms
  if (budget == 0) budget = kHubBudgetDefault;
  const long long max_hubs = budget / (words * 4);
  if (max_hubs <= 0) return TDFS_OK;
  cudaError_t e;
  std::vector<std::pair<int64_t, int32_t>> cand;
  const int64_t min_deg = kHubMinDeg;
  for (int64_t v = 0; v < G.n; v++) {
    int64_t d = offs[v + 1] - offs[v];
    if (d >= min_deg) cand.push_back({-d, (int32_t)v});
  }
  if (cand.empty()) return TDFS_OK;
  if ((long long)cand.size() > max_hubs) {
    std::nth_element(cand.begin(), cand.begin() + max_hubs, cand.end());
    cand.resize(max_hubs);
  }
  std::sort(cand.begin(), cand.end());
  std::vector<int32_t> hub_id((size_t)G.n, -1), hub_vertex(cand.size());
  for (size_t h = 0; h < cand.size(); h++) {
    hub_vertex[h] = cand[h].second;
    hub_id[cand[h].second] = (int32_t)h;
  }
  G.n_hubs = (int64_t)cand.size();
  G.hub_words = words;
  G.hub_min_deg = -cand.back().first;
  int32_t* d_vert = nullptr;
  if ((e = cudaMalloc(&G.d_hub_id, sizeof(int32_t) * G.n)) != cudaSuccess ||
      (e = cudaMalloc(&G.d_hub_bits, sizeof(uint32_t) * (size_t)(G.n_hubs * words))) != cudaSuccess ||
      (e = cudaMalloc(&d_vert, sizeof(int32_t) * G.n_hubs)) != cudaSuccess) {
    cudaFree(d_vert);
    return fail(TDFS_E_OOM, "hubs: alloc");
  }
  cudaMemcpyAsync(G.d_hub_id, hub_id.data(), sizeof(int32_t) * G.n, cudaMemcpyHostToDevice, st);
  cudaMemcpyAsync(d_vert, hub_vertex.data(), sizeof(int32_t) * G.n_hubs, cudaMemcpyHostToDevice, st);
  cudaMemsetAsync(G.d_hub_bits, 0, sizeof(uint32_t) * (size_t)(G.n_hubs * words), st);
  hub_bits_kernel<<<(int)std::min<int64_t>(G.n_hubs, 65535), 256, 0, st>>>(G.d_offs, G.d_adj, d_vert, G.n_hubs, words,
                                                                         G.d_hub_bits);
  e = cudaStreamSynchronize(st);
  cudaFree(d_vert);
  if (e != cudaSuccess) return cuda_fail(e, "hubs: build");
  return TDFS_OK;
}

int build_indexes(Graph& G, cudaStream_t st, int64_t hub_budget) {
  std::vector<int64_t> offs((size_t)G.n + 1);
  cudaError_t e = cudaMemcpyAsync(offs.data(), G.d_offs, sizeof(int64_t) * (G.n + 1), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail(e, "index: offs copy");
  return build_hub_bitmaps(G, st, offs, hub_budget);
}

int finish_device_graph(Graph& G, cudaStream_t st, bool scan_on_device, bool enforce, int64_t hub_budget) {
  cudaError_t e;
  if ((e = cudaMalloc(&G.d_src, sizeof(int32_t) * (size_t)std::max<int64_t>(G.nnz, 1))) != cudaSuccess)
    return fail(TDFS_E_OOM, std::string("load: src array: ") + cudaGetErrorString(e));
  int dev_sms = 148;
  cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, G.device);
  fill_src_kernel<<<dev_sms * 8, 256, 0, st>>>(G.d_offs, G.n, G.d_src);
  if ((e = cudaGetLastError()) != cudaSuccess) return cuda_fail(e, "load: fill_src");
  if (scan_on_device) {
    unsigned long long* d_out = nullptr;
    if ((e = cudaMalloc(&d_out, 3 * sizeof(unsigned long long))) != cudaSuccess) return cuda_fail(e, "load: scan");
    cudaMemsetAsync(d_out, 0, 3 * sizeof(unsigned long long), st);
    scan_graph_kernel<<<dev_sms * 8, 256, 0, st>>>(G.d_offs, G.d_adj, G.d_label, G.n, G.nnz, enforce ? 1 : 0, d_out);
    unsigned long long h[3];
    e = cudaMemcpyAsync(h, d_out, sizeof(h), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaFree(d_out);
    if (e != cudaSuccess) return cuda_fail(e, "load: scan");
    if (h[1] & 2) return fail(TDFS_E_ID_RANGE, "load (device scan): id out of range [0, n)");
    if (enforce && (h[1] & 1)) return fail(TDFS_E_GRAPH_FORMAT, "validate (device): bad CSR (order/dup/self-loop/asymmetric/offs)");
    G.dmax = (int64_t)h[0];
    G.nlabels = G.d_label ? (int32_t)h[2] + 1 : 1;
  }
  if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return cuda_fail(e, "load: sync");
  return build_indexes(G, st, hub_budget);
}

void release(Graph& G) {
  if (G.owns_csr) {
    cudaFree(G.d_offs);
    cudaFree(G.d_adj);
    cudaFree(G.d_label);
  }
  cudaFree(G.d_src);
  cudaFree(G.d_hub_id);
  cudaFree(G.d_hub_bits);
  free_shard_lists(&G);
  cudaFree(G.d_orig);
  G.d_orig = nullptr;
  G.d_offs = nullptr; G.d_adj = nullptr; G.d_label = nullptr; G.d_src = nullptr;
  G.d_hub_id = nullptr; G.d_hub_bits = nullptr; G.n_hubs = 0;
}

int upload(Graph& G, const int64_t* offs, const int32_t* adj, const uint8_t* label, cudaStream_t st);
void host_stats(Graph& G, const int64_t* offs, const uint8_t* label);
void relabel_by_degree(int64_t n, const int64_t* offs, const int32_t* adj, const uint8_t* label,
                       std::vector<int64_t>& noffs, std::vector<int32_t>& nadj, std::vector<uint8_t>& nlabel,
                       std::vector<int32_t>& orig);

// Host CSR (already simple, symmetric, sorted) -> device, optionally relabelled by degree, then the
// per-entry sources and hub bitmaps.  Synchronous (host vectors outlive the copies).
int finish_host_csr(Graph& G, const int64_t* offs, const int32_t* adj, const uint8_t* label, uint32_t flags,
                    int64_t hub_budget, cudaStream_t st) {
  std::vector<int64_t> noffs;
  std::vector<int32_t> nadj, orig;
  std::vector<uint8_t> nlabel;
  if (flags & TDFS_GRAPH_DEGREE_ORDER) {
    relabel_by_degree(G.n, offs, adj, label, noffs, nadj, nlabel, orig);
    offs = noffs.data();
    adj = nadj.data();
    if (label) label = nlabel.data();
  }
  host_stats(G, offs, label);
  int rc = upload(G, offs, adj, label, st);
  if (rc == TDFS_OK && !orig.empty()) {
    cudaError_t e = cudaMalloc(&G.d_orig, sizeof(int32_t) * orig.size());
    if (e == cudaSuccess) e = cudaMemcpyAsync(G.d_orig, orig.data(), sizeof(int32_t) * orig.size(), cudaMemcpyHostToDevice, st);
    if (e != cudaSuccess) rc = fail(TDFS_E_OOM, "load: degree-order map");
  }
  if (rc == TDFS_OK) rc = finish_device_graph(G, st, false, false, hub_budget);
  return rc;
}

int upload(Graph& G, const int64_t* offs, const int32_t* adj, const uint8_t* label, cudaStream_t st) {
  cudaError_t e;
  G.owns_csr = true;
  size_t bo = sizeof(int64_t) * (size_t)(G.n + 1), ba = sizeof(int32_t) * (size_t)std::max<int64_t>(G.nnz, 1);
  if ((e = cudaMalloc(&G.d_offs, bo)) != cudaSuccess) return fail(TDFS_E_OOM, "load: offs alloc");
  if ((e = cudaMalloc(&G.d_adj, ba)) != cudaSuccess) return fail(TDFS_E_OOM, "load: adj alloc");
  if (label && (e = cudaMalloc(&G.d_label, (size_t)std::max<int64_t>(G.n, 1))) != cudaSuccess)
    return fail(TDFS_E_OOM, "load: label alloc");
  if ((e = cudaMemcpyAsync(G.d_offs, offs, bo, cudaMemcpyHostToDevice, st)) != cudaSuccess) return cuda_fail(e, "load: offs copy");
  if (G.nnz && (e = cudaMemcpyAsync(G.d_adj, adj, sizeof(int32_t) * (size_t)G.nnz, cudaMemcpyHostToDevice, st)) != cudaSuccess)
    return cuda_fail(e, "load: adj copy");
  if (label && G.n && (e = cudaMemcpyAsync(G.d_label, label, (size_t)G.n, cudaMemcpyHostToDevice, st)) != cudaSuccess)
    return cuda_fail(e, "load: label copy");
  return TDFS_OK;
}

// TDFS_GRAPH_DEGREE_ORDER (R35): vertex r of the device graph is the user's vertex orig[r], where
// the user's vertices are sorted by (degree, id); lists are re-sorted in the new ids.  Symmetry-breaking
// constraints then compare degree ranks, so the lower-ranked (lower-degree) vertex roots each copy.
void relabel_by_degree(int64_t n, const int64_t* offs, const int32_t* adj, const uint8_t* label,
                       std::vector<int64_t>& noffs, std::vector<int32_t>& nadj, std::vector<uint8_t>& nlabel,
                       std::vector<int32_t>& orig) {
  orig.resize((size_t)n);
  for (int64_t v = 0; v < n; v++) orig[v] = (int32_t)v;
  std::stable_sort(orig.begin(), orig.end(), [&](int32_t a, int32_t b) {
    return offs[a + 1] - offs[a] < offs[b + 1] - offs[b];
  });
  std::vector<int32_t> rank((size_t)n);
  for (int64_t r = 0; r < n; r++) rank[orig[r]] = (int32_t)r;
  noffs.assign((size_t)n + 1, 0);
  for (int64_t r = 0; r < n; r++) noffs[r + 1] = noffs[r] + (offs[orig[r] + 1] - offs[orig[r]]);
  nadj.resize((size_t)noffs[n]);
  parallel_for(n, [&](int64_t lo, int64_t hi) {
    for (int64_t r = lo; r < hi; r++) {
      const int32_t v = orig[r];
      int32_t* L = nadj.data() + noffs[r];
      const int64_t d = offs[v + 1] - offs[v];
      for (int64_t i = 0; i < d; i++) L[i] = rank[adj[offs[v] + i]];
      std::sort(L, L + d);
    }
  });
  if (label) {
    nlabel.resize((size_t)n);
    for (int64_t r = 0; r < n; r++) nlabel[r] = label[orig[r]];
  }
}

void host_stats(Graph& G, const int64_t* offs, const uint8_t* label) {
  int64_t dmax = 0;
  for (int64_t v = 0; v < G.n; v++) dmax = std::max(dmax, offs[v + 1] - offs[v]);
  G.dmax = dmax;
  int lmax = 0;
  if (label)
    for (int64_t v = 0; v < G.n; v++) lmax = std::max(lmax, (int)label[v]);
  G.nlabels = lmax + 1;
}

}  // namespace

const Graph* graph_of(const tdfs_graph* g) { return g ? &g->g : nullptr; }

}  // namespace tdfs

using namespace tdfs;

extern "C" int tdfs_load_graph(const tdfs_csr* c, int device, void* stream, tdfs_graph** out) {
  if (!c || !out) return fail(TDFS_E_INVALID_ARG, "load_graph: NULL argument");
  if (c->n < 0 || c->nnz < 0 || !c->offs || (c->nnz > 0 && !c->adj)) return fail(TDFS_E_INVALID_ARG, "load_graph: bad CSR");
  if (c->n >= kMaxN) return fail(TDFS_E_ID_RANGE, "load_graph: n >= 2^31 - 2");
  if (c->mem != TDFS_MEM_HOST_COPY && c->mem != TDFS_MEM_DEVICE_BORROW) return fail(TDFS_E_INVALID_ARG, "load_graph: bad mem");
  if (c->mem == TDFS_MEM_DEVICE_BORROW && (c->flags & (TDFS_GRAPH_NORMALIZE | TDFS_GRAPH_DEGREE_ORDER)))
    return fail(TDFS_E_INVALID_ARG, "load_graph: NORMALIZE / DEGREE_ORDER need HOST_COPY");
  if (c->flags & ~(TDFS_GRAPH_VALIDATE | TDFS_GRAPH_NORMALIZE | TDFS_GRAPH_DEGREE_ORDER))
    return fail(TDFS_E_INVALID_ARG, "load_graph: unknown flags");
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) return cuda_fail(e, "load_graph: cudaSetDevice");
  cudaStream_t st = (cudaStream_t)stream;
  tdfs_graph* h = new (std::nothrow) tdfs_graph;
  if (!h) return fail(TDFS_E_OOM, "load_graph: host alloc");
  Graph& G = h->g;
  G.device = device;
  G.n = c->n;
  int rc = TDFS_OK;
  if (c->mem == TDFS_MEM_HOST_COPY) {
    if (c->flags & TDFS_GRAPH_NORMALIZE) {
      // expand to directed pairs, then symmetric simple CSR
      for (int64_t v = 0; v < c->n; v++)
        if (c->offs[v + 1] < c->offs[v]) { delete h; return fail(TDFS_E_GRAPH_FORMAT, "load_graph: offsets decrease"); }
      if (c->offs[0] != 0 || c->offs[c->n] != c->nnz) { delete h; return fail(TDFS_E_GRAPH_FORMAT, "load_graph: offs/nnz mismatch"); }
      std::vector<int32_t> a((size_t)c->nnz);
      for (int64_t v = 0; v < c->n; v++)
        for (int64_t i = c->offs[v]; i < c->offs[v + 1]; i++) {
          if (c->adj[i] < 0 || c->adj[i] >= c->n) { delete h; return fail(TDFS_E_ID_RANGE, "load_graph: id out of range"); }
          a[i] = (int32_t)v;
        }
      std::vector<int64_t> offs;
      std::vector<int32_t> adj;
      build_csr(c->n, c->nnz, a.data(), c->adj, offs, adj);
      G.nnz = offs[c->n];
      rc = finish_host_csr(G, offs.data(), adj.data(), c->label, c->flags, c->hub_bitmap_bytes, st);
    } else {
      if (c->flags & TDFS_GRAPH_VALIDATE) rc = validate_host(c->n, c->nnz, c->offs, c->adj);
      else rc = check_host_ids(c->n, c->nnz, c->offs, c->adj);  // cheap: ids in [0, n), offsets sane
      G.nnz = c->nnz;
      if (rc == TDFS_OK) rc = finish_host_csr(G, c->offs, c->adj, c->label, c->flags, c->hub_bitmap_bytes, st);
    }
  } else {
    G.owns_csr = false;
    G.nnz = c->nnz;
    G.d_offs = const_cast<int64_t*>(c->offs);
    G.d_adj = const_cast<int32_t*>(c->adj);
    G.d_label = const_cast<uint8_t*>(c->label);
    // d_max and the label count come from a device scan; VALIDATE adds the format checks
    rc = finish_device_graph(G, st, true, (c->flags & TDFS_GRAPH_VALIDATE) != 0, c->hub_bitmap_bytes);
  }
  if (rc != TDFS_OK) {
    release(G);
    delete h;
    return rc;
  }
  *out = h;
  return TDFS_OK;
}

extern "C" int tdfs_load_edges(int64_t n, int64_t m, const int32_t* src, const int32_t* dst, const uint8_t* label,
                               uint32_t flags, int64_t hub_bitmap_bytes, int device, void* stream, tdfs_graph** out) {
  if (!out || n < 0 || m < 0 || (m > 0 && (!src || !dst))) return fail(TDFS_E_INVALID_ARG, "load_edges: bad args");
  if (flags & ~(uint32_t)TDFS_GRAPH_DEGREE_ORDER) return fail(TDFS_E_INVALID_ARG, "load_edges: flags other than DEGREE_ORDER");
  if (n >= kMaxN) return fail(TDFS_E_ID_RANGE, "load_edges: n >= 2^31 - 2");
  std::atomic<int> bad(0);
  parallel_for(m, [&](int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; i++)
      if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n) { bad = 1; return; }
  });
  if (bad.load()) return fail(TDFS_E_ID_RANGE, "load_edges: endpoint outside [0, n)");
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) return cuda_fail(e, "load_edges: cudaSetDevice");
  cudaStream_t st = (cudaStream_t)stream;
  std::vector<int64_t> offs;
  std::vector<int32_t> adj;
  build_csr(n, m, src, dst, offs, adj);
  tdfs_graph* h = new (std::nothrow) tdfs_graph;
  if (!h) return fail(TDFS_E_OOM, "load_edges: host alloc");
  Graph& G = h->g;
  G.device = device;
  G.n = n;
  G.nnz = offs[n];
  int rc = finish_host_csr(G, offs.data(), adj.data(), label, flags, hub_bitmap_bytes, st);
  if (rc != TDFS_OK) {
    release(G);
    delete h;
    return rc;
  }
  *out = h;
  return TDFS_OK;
}

extern "C" int tdfs_graph_info(const tdfs_graph* g, int64_t* n, int64_t* m, int64_t* dmax, int32_t* nlabels) {
  if (!g) return fail(TDFS_E_INVALID_ARG, "graph_info: NULL graph");
  if (n) *n = g->g.n;
  if (m) *m = g->g.nnz / 2;
  if (dmax) *dmax = g->g.dmax;
  if (nlabels) *nlabels = g->g.nlabels;
  return TDFS_OK;
}

extern "C" int tdfs_graph_device_arrays(const tdfs_graph* g, const int64_t** offs, const int32_t** adj,
                                        const uint8_t** label) {
  if (!g) return fail(TDFS_E_INVALID_ARG, "graph_device_arrays: NULL graph");
  if (offs) *offs = g->g.d_offs;
  if (adj) *adj = g->g.d_adj;
  if (label) *label = g->g.d_label;
  return TDFS_OK;
}

extern "C" void tdfs_free_graph(tdfs_graph* g) {
  if (!g) return;
  cudaSetDevice(g->g.device);
  release(g->g);
  delete g;
}
