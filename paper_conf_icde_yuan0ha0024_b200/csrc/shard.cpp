// Multi-GPU plumbing of libtdfs.so:
//  - the partition of the initial edge tasks over ranks (tdfs_partition_edges and the per-rank
//    device task lists used by tdfs_count with shard_policy = TDFS_SHARD_DEGREE_BALANCED);
//  - a chunk cursor in one GPU's memory that other ranks map through CUDA IPC, so that every
//    rank's persistent kernel takes edge chunks from one shared counter (cross-GPU dynamic
//    balancing; the paper deals edges round-robin and does no migration).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <numeric>
#include <vector>

#include "internal.h"

namespace tdfs {

// Owner rank of every directed edge (CSR index e).
//  ROUND_ROBIN: e mod W.
//  DEGREE_BALANCED (R31, north_star "root-vertex tasks (degree-balanced)"): the cost of
//  a root v is c(v) = sum over w in N(v) of deg(w) (the adjacency a root's edge tasks intersect
//  with at the next level).  A root with c(v) > C / (64 W) (C = total cost) is too coarse to be
//  dealt whole: its edges are dealt round-robin (edge granularity, as in the paper).  The other
//  roots are dealt whole, in decreasing cost, in snake order over the ranks (0..W-1, W-1..0, ...)
//  so that every round of W roots adds about the same cost to every rank.
int partition_owner(int64_t n, int64_t nnz, const int64_t* offs, const int32_t* adj, int world, int policy,
                    int32_t* owner) {
  if (world < 1) return fail(TDFS_E_INVALID_ARG, "partition: world < 1");
  if (n < 0 || nnz < 0 || !offs || (nnz > 0 && (!adj || !owner))) return fail(TDFS_E_INVALID_ARG, "partition: bad CSR");
  if (policy == TDFS_SHARD_ROUND_ROBIN) {
    for (int64_t e = 0; e < nnz; e++) owner[e] = (int32_t)(e % world);
    return TDFS_OK;
  }
  if (policy == TDFS_SHARD_BLOCKED) {
    for (int64_t e = 0; e < nnz; e++) owner[e] = (int32_t)((e / TDFS_SHARD_BLOCK_EDGES) % world);
    return TDFS_OK;
  }
  if (policy != TDFS_SHARD_DEGREE_BALANCED) return fail(TDFS_E_INVALID_ARG, "partition: unknown policy");
  if (nnz >= (int64_t)INT32_MAX) return fail(TDFS_E_INVALID_ARG, "partition: nnz >= 2^31 (degree-balanced lists are int32)");
  if (offs[0] != 0 || offs[n] != nnz) return fail(TDFS_E_INVALID_ARG, "partition: offs[0] != 0 or offs[n] != nnz");
  std::vector<int64_t> cost((size_t)n, 0);
  long double total = 0;
  for (int64_t v = 0; v < n; v++) {
    int64_t c = 0;
    for (int64_t e = offs[v]; e < offs[v + 1]; e++) {
      const int32_t w = adj[e];
      if (w < 0 || w >= n) return fail(TDFS_E_ID_RANGE, "partition: id out of range");
      c += offs[w + 1] - offs[w];
    }
    cost[v] = c;
    total += (long double)c;
  }
  const long double heavy = total / (64.0L * world);
  std::vector<int32_t> light;
  int64_t rr = 0;  // running index over heavy roots' edges
  for (int64_t v = 0; v < n; v++) {
    if (offs[v + 1] == offs[v]) continue;
    if ((long double)cost[v] > heavy) {
      for (int64_t e = offs[v]; e < offs[v + 1]; e++) owner[e] = (int32_t)(rr++ % world);
    } else {
      light.push_back((int32_t)v);
    }
  }
  std::stable_sort(light.begin(), light.end(), [&](int32_t a, int32_t b) { return cost[a] > cost[b]; });
  for (size_t i = 0; i < light.size(); i++) {
    const int64_t round = (int64_t)i / world, t = (int64_t)i % world;
    const int32_t r = (int32_t)((round & 1) ? world - 1 - t : t);
    const int32_t v = light[i];
    for (int64_t e = offs[v]; e < offs[v + 1]; e++) owner[e] = r;
  }
  return TDFS_OK;
}

// Device list of the directed edges of `rank` (ascending CSR index), cached on the graph.
int shard_task_list(const Graph* g, int rank, int world, int policy, const int32_t** d_tasks, int64_t* n_tasks) {
  for (const auto& s : g->shard_lists)
    if (s.rank == rank && s.world == world) {
      *d_tasks = s.d_tasks;
      *n_tasks = s.n;
      return TDFS_OK;
    }
  std::vector<int64_t> offs((size_t)g->n + 1);
  std::vector<int32_t> adj((size_t)std::max<int64_t>(g->nnz, 1));
  cudaError_t e = cudaMemcpy(offs.data(), g->d_offs, sizeof(int64_t) * (size_t)(g->n + 1), cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && g->nnz)
    e = cudaMemcpy(adj.data(), g->d_adj, sizeof(int32_t) * (size_t)g->nnz, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return fail(TDFS_E_CUDA, std::string("shard list: ") + cudaGetErrorString(e));
  std::vector<int32_t> owner((size_t)std::max<int64_t>(g->nnz, 1));
  int rc = partition_owner(g->n, g->nnz, offs.data(), adj.data(), world, policy, owner.data());
  if (rc) return rc;
  std::vector<int32_t> mine;
  for (int64_t i = 0; i < g->nnz; i++)
    if (owner[i] == rank) mine.push_back((int32_t)i);
  int32_t* d = nullptr;
  if ((e = cudaMalloc(&d, sizeof(int32_t) * std::max<size_t>(mine.size(), 1))) != cudaSuccess)
    return fail(TDFS_E_OOM, "shard list: alloc");
  if (!mine.empty() &&
      (e = cudaMemcpy(d, mine.data(), sizeof(int32_t) * mine.size(), cudaMemcpyHostToDevice)) != cudaSuccess) {
    cudaFree(d);
    return fail(TDFS_E_CUDA, std::string("shard list: ") + cudaGetErrorString(e));
  }
  g->shard_lists.push_back({rank, world, d, (int64_t)mine.size()});
  *d_tasks = d;
  *n_tasks = (int64_t)mine.size();
  return TDFS_OK;
}

void free_shard_lists(const Graph* g) {
  for (auto& s : g->shard_lists) cudaFree(s.d_tasks);
  g->shard_lists.clear();
}

}  // namespace tdfs

using namespace tdfs;

extern "C" int tdfs_partition_edges(int64_t n, int64_t nnz, const int64_t* offs, const int32_t* adj, int32_t world,
                                    int32_t policy, int32_t* owner) {
  return partition_owner(n, nnz, offs, adj, world, policy, owner);
}

static_assert(sizeof(cudaIpcMemHandle_t) == 64, "cudaIpcMemHandle_t is 64 bytes");

extern "C" int tdfs_shared_cursor_create(int device, uint64_t** d_cursor, void* ipc_handle) {
  if (!d_cursor || !ipc_handle) return fail(TDFS_E_INVALID_ARG, "shared_cursor_create: NULL");
  cudaError_t e = cudaSetDevice(device);
  void* p = nullptr;
  if (e == cudaSuccess) e = cudaMalloc(&p, 256);  // own 256-byte line
  if (e != cudaSuccess) return fail(TDFS_E_OOM, std::string("shared_cursor_create: ") + cudaGetErrorString(e));
  cudaIpcMemHandle_t h;
  if ((e = cudaMemset(p, 0, 256)) != cudaSuccess || (e = cudaIpcGetMemHandle(&h, p)) != cudaSuccess) {
    cudaFree(p);
    return fail(TDFS_E_CUDA, std::string("shared_cursor_create: ") + cudaGetErrorString(e));
  }
  std::memcpy(ipc_handle, &h, sizeof(h));
  *d_cursor = static_cast<uint64_t*>(p);
  return TDFS_OK;
}

extern "C" int tdfs_shared_cursor_open(int device, const void* ipc_handle, uint64_t** d_cursor) {
  if (!d_cursor || !ipc_handle) return fail(TDFS_E_INVALID_ARG, "shared_cursor_open: NULL");
  cudaError_t e = cudaSetDevice(device);
  cudaIpcMemHandle_t h;
  std::memcpy(&h, ipc_handle, sizeof(h));
  void* p = nullptr;
  if (e == cudaSuccess) e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) return fail(TDFS_E_CUDA, std::string("shared_cursor_open: ") + cudaGetErrorString(e));
  *d_cursor = static_cast<uint64_t*>(p);
  return TDFS_OK;
}

extern "C" int tdfs_shared_cursor_reset(uint64_t* d_cursor, void* stream) {
  if (!d_cursor) return fail(TDFS_E_INVALID_ARG, "shared_cursor_reset: NULL");
  cudaError_t e = cudaMemsetAsync(d_cursor, 0, sizeof(uint64_t), (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(TDFS_E_CUDA, std::string("shared_cursor_reset: ") + cudaGetErrorString(e));
  return TDFS_OK;
}

extern "C" int tdfs_shared_cursor_close(uint64_t* d_cursor, int opened) {
  if (!d_cursor) return TDFS_OK;
  cudaError_t e = opened ? cudaIpcCloseMemHandle(d_cursor) : cudaFree(d_cursor);
  if (e != cudaSuccess) return fail(TDFS_E_CUDA, std::string("shared_cursor_close: ") + cudaGetErrorString(e));
  return TDFS_OK;
}
