// Internal declarations of libtdfs.so (not part of the ABI).
#pragma once

#include <cstddef>
#include <cstdint>
#include <string>
#include <vector>

#include "tdfs.h"

namespace tdfs {

constexpr int kMaxK = TDFS_MAX_K;

// ---------------------------------------------------------------- errors
void set_error(const std::string& msg);
int fail(int status, const std::string& msg);  // sets the detail, returns status

// ---------------------------------------------------------------- plan
// Per matching-order position p (pi_p = order[p]) everything the kernel needs,
// precomputed on the host (PAPER.md:77 backward neighbours, :29 constraints,
// :400 degree/label filters).  Bit j of a mask refers to position j < p.
// Index kVF of the per-position arrays is a VIRTUAL position: the part of the last
// position's Eq. (1) that does not depend on S[k-2] -- the "fixed" operands
// B(u_{k-1}) restricted to positions <= k-3, the constraint windows and injectivity
// tests against those positions, and the label/degree filters.  Its result F is
// the same for every sibling at level k-2, so it is computed once per level-(k-2)
// list and staged in shared memory; each leaf is then
// |F ∩ N(S[k-2])| (or |F| minus S[k-2]) under the S[k-2]-dependent window.
constexpr int kVF = kMaxK;
constexpr int kBlockThreads = 128;  // matching-kernel block size (its __launch_bounds__)
#ifndef TDFS_LEAF_STAGE_MAX  // build-time constant (experiments build variants with -D)
#define TDFS_LEAF_STAGE_MAX 512
#endif
constexpr int kLeafStage = TDFS_LEAF_STAGE_MAX;  // shared-memory ids per warp for a materialised leaf set F (at most)
// Hub bitmaps (graph.cu): vertices of degree >= kHubMinDeg, highest first, within the budget
constexpr int64_t kHubMinDeg = 256;
constexpr int64_t kHubBudgetDefault = 256ll << 20;
// Eq. (1) / leaf-batch cost model (measured on config 2; fixed, no run-time knobs)
constexpr int kMergeRatio = 4;      // probe by warp merge when |B| <= 4 |A remaining|, else binary search
constexpr int kUaHub = 4;           // stream A: per-element cost of probing a hub bitmap of N(x)
constexpr int kUbRef = 4;           // stream B: per-element cost of probing a referenced F's bitmap
constexpr int kRangeMin = 32;       // range tasks: >= 32 siblings each ...
constexpr int kRangeMaxT = 32;      // ... and <= 32 tasks per split
struct DevPlan {
  int32_t k;
  int32_t order[kMaxK];          // query vertex at position p (enumerate output mapping)
  uint32_t bwd[kMaxK + 1];       // B^pi(pi_p) as a position mask
  uint32_t lo_mask[kMaxK + 1];   // j with constraint f(pi_j) < f(pi_p): v > S[j]
  uint32_t hi_mask[kMaxK + 1];   // j with constraint f(pi_p) < f(pi_j): v < S[j]
  uint32_t inj_mask[kMaxK + 1];  // j whose v != S[j] is not implied by adjacency or a constraint
  int32_t label[kMaxK + 1];      // required label, -1 = any
  int32_t deg_min[kMaxK + 1];    // degree filter threshold (0 = off), R8
  int32_t edge_cons;             // constraint between positions 0 and 1: +1 S0<S1, -1 S1<S0, 0 none
  int32_t reuse_enabled;         // set-intersection result reuse on
  int8_t reuse[kMaxK + 1];       // stored position r whose candidate list C(r) is a superset start for p, -1 none
  uint8_t shortcut[kMaxK + 1];   // last position: count without scanning; bit0 valid with reuse, bit1 without
  // roofline bytes (R32, STATS only): stored positions r whose C(r) may serve as an Eq. (1)
  // source of p (every reuse candidate, not only the chosen one), and "p is count-only"
  uint32_t src_mask[kMaxK + 1];
  uint8_t cnt_only[kMaxK + 1];
  // leaf staging (position k-1 split into the virtual position kVF and the S[k-2] part)
  int8_t lf_on;                  // k >= 4 and B(u_{k-1}) has an operand at a position <= k-3
  int8_t lf_var;                 // N(S[k-2]) is an operand of position k-1
  int8_t lf_lo_var, lf_hi_var;   // window bound v > S[k-2] / v < S[k-2]
  int8_t lf_inj_var;             // v != S[k-2] must be tested (not implied)
  int8_t lf_byref;               // F = a window of one adjacency list, no per-element filter (FRef by reference)
};

struct Plan {
  int k = 0;
  std::vector<std::pair<int, int>> qedges;
  std::vector<int> qlabel;   // empty = unlabeled
  std::vector<int> order;
  std::vector<std::pair<int, int>> constraints;
  int64_t n_aut = 1;
  DevPlan dev{};
};

// ---------------------------------------------------------------- graph
struct Graph {
  int device = 0;
  int64_t n = 0, nnz = 0, dmax = 0;
  int32_t nlabels = 1;
  int64_t* d_offs = nullptr;
  int32_t* d_adj = nullptr;
  uint8_t* d_label = nullptr;
  int32_t* d_src = nullptr;  // source vertex of each directed entry (edge tasks)
  int32_t* d_orig = nullptr; // TDFS_GRAPH_DEGREE_ORDER: user id of device vertex r (nullptr = identity)
  bool owns_csr = true;
  // hub adjacency bitmaps: membership w in N(h) in O(1) for the highest-degree vertices
  int32_t* d_hub_id = nullptr;     // [n], -1 for non-hubs
  uint32_t* d_hub_bits = nullptr;  // [n_hubs][hub_words]
  int64_t n_hubs = 0, hub_words = 0, hub_min_deg = 0;
  // degree-balanced shard task lists, built on first use per (rank, world) (shard.cpp)
  struct ShardList { int32_t rank, world; int32_t* d_tasks; int64_t n; };
  mutable std::vector<ShardList> shard_lists;
};

// ---------------------------------------------------------------- device job
// One task of Q_task, 32 bytes (one sector; PAPER.md:191 uses 3 ints).  hdr = kind | level << 4:
//   TASK_EDGE    <v1, v2>              an initial edge task (PAPER.md:189 <v1,v2,-2>), DFS from level 2
//   TASK_PREFIX  <v1, v2, v3>          a 3-prefix task, DFS from level 3
//   TASK_RANGE   <S0 .. S_{d-1}, lo, hi>  level d (2 <= d <= 4) candidates of that prefix with ids in
//                                      [lo, hi) (R30/R33 range tasks), DFS from level d
constexpr int TASK_EDGE = 0, TASK_PREFIX = 1, TASK_RANGE = 2;
constexpr int kMaxRangeLevel = 4;  // d + 2 ints (prefix, lo, hi) fit the 6 payload words
struct QSlot {
  int32_t hdr;
  int32_t v[6];
  uint32_t seq;               // ticket handshake: == t free for ticket t, == t+1 full for ticket t
};
static_assert(sizeof(QSlot) == 32, "one 32-byte sector per task");

enum CounterIdx {            // each counter on its own 128-byte line
  C_COUNT = 0, C_CURSOR, C_QHEAD, C_QTAIL, C_QAVAIL, C_QFREE, C_ACTIVE, C_POOL, C_ERROR, C_OUTCUR, C_TRACE,
  C_CONSUMED,                  // streaming enumerate: tuples the host has drained (written by the host)
  C_NUM
};
constexpr int kCounterStride = 16;  // u64 words per counter (128 B)

enum StatIdx {
  S_NODES = 0,                 // 9 entries
  S_ADJ_BYTES = 9, S_ENQ, S_DEQ, S_TIMEOUTS, S_QFULL, S_EDGES_SCANNED, S_EDGES_IN, S_CHUNKS, S_STREAM,
  S_T_START,                   // min over warps of the start time (%globaltimer ns)
  S_T_EXIT_MIN, S_T_EXIT_MAX, S_T_EXIT_SUM, S_WARPS,  // warp exit times (absolute ns; sum over warps)
  S_NUM
};

struct KParams {
  // graph
  const int64_t* offs;
  const int32_t* adj;
  const int32_t* src;
  const uint8_t* label;
  int64_t n;
  // plan
  DevPlan plan;
  // initial tasks: this shard's directed edges e = shard_rank + j * shard_world
  int64_t n_tasks;             // number of j
  int32_t shard_rank, shard_world;
  int32_t chunk;
  int32_t n_levels;            // stored stack levels = max(0, k - 3): positions 2 .. k-2
  // queue
  QSlot* slots;
  uint64_t qcap;                // capacity in tasks (initial value of the `free` counter)
  uint64_t qslots;              // ring slots: next power of two >= qcap (index = ticket & (qslots - 1))
  // counters
  unsigned long long* ctr;     // C_NUM * kCounterStride u64
  unsigned long long* stats;   // S_NUM u64 or nullptr
  // paged stacks (Alg. 5)
  uint32_t* page_tables;       // [n_warps][n_levels][E], 0xFFFFFFFF = null
  int32_t* pool;               // n_pages pages of (1 << page_shift) ints
  uint32_t n_pages;
  int32_t page_shift;          // log2(ints per page)
  int32_t E;                   // page-table entries per level
  int32_t array_stacks;        // ablation: contiguous per-warp-level arrays of E pages (identity page tables)
  int64_t tau_ns;              // < 0: infinity
  int32_t fcap;                // leaf staging: shared-memory ids per warp (0 = off)
  int32_t meta_off;            // shared-memory layout: byte offset of the warps' leaf-batch entries
  uint32_t split_mask;         // bit d: level d is split-eligible -- 2 (the paper's rule) and the
                               // range-task levels up to kMaxRangeLevel (R33)
  uint32_t range_mask;         // bit d: a timed-out level d splits into <= 32 id-range tasks (R30/R33); level 2
                               // without the bit pushes one <S0,S1,v> task per sibling
  uint32_t reused_mask;        // bit d: a later position / the leaf set reuses C(d) (range tasks then build it whole)
  // initial edge tasks: j -> directed edge task_edges[j] (shard list) or shard_rank + j * shard_world
  const int32_t* task_edges;   // nullptr = arithmetic shard
  int32_t shard_block;         // arithmetic shard: 0 = edge round-robin (e = rank + j W), else blocks of this many
                               // consecutive edges dealt round-robin (TDFS_SHARD_BLOCKED)
  unsigned long long* gcursor; // chunk cursor: this job's counter, or a cross-rank shared one (NEXT-3)
  int32_t gshared;             // gcursor is shared across ranks / devices: system-scope atomics
  // hub bitmaps (nullptr when off)
  const int32_t* hub_id;
  const uint32_t* hub_bits;
  long long hub_words;
  // enumerate
  const int32_t* orig;             // device id -> user id (degree-ordered graphs), nullptr = identity
  int32_t* out;
  unsigned long long cap;
  unsigned long long ring_chunk;   // streaming (NEXT-2): tuples per ring chunk, 0 = capacity mode
  unsigned long long ring_nchunks;
  unsigned long long* ring_fill;   // [ring_nchunks] tuples written into each chunk (reset by the host)
  // tracing (tests)
  int32_t* trace;
  long long trace_cap;
};

// workspace layout (byte offsets from the 256-aligned base)
constexpr int kRingChunks = 8;  // streaming enumerate: the output ring is drained in 8 chunks
struct WsLayout {
  size_t ctr = 0, stats = 0, fill = 0, slots = 0, tables = 0, pool = 0, total = 0;
  uint64_t qcap = 0, qslots = 0, n_pages = 0;
  int32_t E = 0, page_shift = 0, n_levels = 0, blocks = 0, wpb = 0, fcap = 0;
};

int resolve_layout(const Graph* g, const Plan* p, const tdfs_run_opts* o, WsLayout* L);
int launch_job(const Graph* g, const Plan* p, const tdfs_run_opts* o, void* ws, size_t ws_bytes, void* stream,
               int mode /*0 count, 1 enumerate*/, int32_t* d_out, uint64_t cap, uint64_t* d_count,
               bool sync, uint64_t* h_count, tdfs_stats* stats, int32_t* h_trace, int64_t trace_cap,
               int64_t* n_trace, bool ring = false);
// streaming enumerate (match.cu): launch in ring mode, then drain chunks to sink until the job ends
typedef int (*SinkFn)(const int32_t* tuples, uint64_t n, int32_t k, void* user);
int stream_job(const Graph* g, const Plan* p, const tdfs_run_opts* o, void* ws, size_t ws_bytes, void* stream,
               int32_t* d_ring, uint64_t ring_cap, SinkFn sink, void* user, uint64_t* n_total);
int blocks_per_sm(int device, int wpb, bool stats, bool enumerate, int fcap, int* out);
const Graph* graph_of(const tdfs_graph* g);
// host partition of the directed edges (tdfs_partition_edges) and the device task list of one rank
int partition_owner(int64_t n, int64_t nnz, const int64_t* offs, const int32_t* adj, int world, int policy,
                    int32_t* owner);
int shard_task_list(const Graph* g, int rank, int world, int policy, const int32_t** d_tasks, int64_t* n_tasks);
void free_shard_lists(const Graph* g);
const Plan* plan_of(const tdfs_plan* p);

}  // namespace tdfs
