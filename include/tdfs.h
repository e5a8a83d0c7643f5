/*
 * tdfs.h -- C-ABI of libtdfs.so, the B200 (sm_100a) hot path of T-DFS
 * ("Faster Depth-First Subgraph Matching on GPUs", Yuan et al., ICDE 2024;
 * /root/reference/PAPER.md, cited below as PAPER.md:<line>).
 *
 * Problem (Section I; Algorithm 1 at PAPER.md:54-73): given an
 * undirected data graph G = (V, E, L) and a query G_Q = (V_Q, E_Q, L_Q), count
 * or enumerate the injective, edge- and label-preserving maps f: V_Q -> V that
 * satisfy a set C of symmetry-breaking constraints f(a) < f(b):
 *
 *   M(G, Q, C) = { f injective | (u,u') in E_Q => {f(u), f(u')} in E;
 *                  L(f(u)) = L_Q(u) when Q is labeled; (a,b) in C => f(a) < f(b) }
 *
 * Matching is non-induced (reading R1).  With the automatic constraint
 * set (full symmetry breaking, R3) every subgraph of G isomorphic to Q
 * is counted exactly once; with no constraints every embedding is counted.
 *
 * Conventions for every entry point:
 *  - returns a tdfs_status (0 = TDFS_OK); never aborts or exits the process;
 *    output arguments are left untouched on error; tdfs_last_error() gives a
 *    thread-local, human-readable detail of the last failure on this thread.
 *  - all ids are 0-based; data vertex ids must satisfy 0 <= id < 2^31 - 2
 *    (-1 and -2 are task-queue sentinels);
 *  - query size k is 2..8 (TDFS_MAX_K); queries must be connected;
 *  - "device" pointers are CUDA global-memory pointers on the graph's device;
 *    "stream" is a cudaStream_t (NULL = legacy default stream).
 *  - No CPU fallback exists: every count is produced by the CUDA kernels.
 */
#ifndef TDFS_H_
#define TDFS_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define TDFS_ABI_VERSION 2
#define TDFS_MAX_K 8

typedef enum {
  TDFS_OK = 0,
  TDFS_E_INVALID_ARG = 1,         /* NULL/negative/inconsistent argument */
  TDFS_E_GRAPH_FORMAT = 2,        /* VALIDATE failed: unsorted, duplicate, self-loop, asymmetric, bad offsets */
  TDFS_E_ID_RANGE = 3,            /* n >= 2^31 - 2 or an id outside [0, n) */
  TDFS_E_QUERY_DISCONNECTED = 4,  /* query (or a user order prefix) not connected */
  TDFS_E_QUERY_TOO_LARGE = 5,     /* k > 8 (or k < 2) */
  TDFS_E_LABEL_RANGE = 6,         /* query label outside [0, 255] */
  TDFS_E_OOM = 7,                 /* device or host allocation failed */
  TDFS_E_STACK_EXHAUSTED = 8,     /* page pool or page table exhausted: NO count is returned */
  TDFS_E_OUTPUT_OVERFLOW = 9,     /* enumerate: more matches than cap; *n_total is still exact */
  TDFS_E_CUDA = 10,               /* a CUDA runtime error (detail in tdfs_last_error) */
  TDFS_E_WORKSPACE = 11           /* workspace NULL, misaligned (256 B) or smaller than tdfs_workspace_bytes */
} tdfs_status;

/* Sentinel written to *d_count by an asynchronous tdfs_count whose kernel failed. */
#define TDFS_COUNT_INVALID (~(uint64_t)0)

const char* tdfs_status_string(int status);
const char* tdfs_last_error(void);
int tdfs_abi_version(void);

/* ------------------------------------------------------------------ graph
 * CSR data graph (Section III: "G is stored in the device memory
 * using the compressed sparse row (CSR) format"), 32-bit vertex ids
 * (PAPER.md:350), optional vertex labels.
 */
typedef struct tdfs_graph tdfs_graph; /* opaque, library-owned */

#define TDFS_MEM_HOST_COPY 0      /* offs/adj/label are host arrays, copied to library-owned device memory */
#define TDFS_MEM_DEVICE_BORROW 1  /* offs/adj/label are device arrays; caller keeps them alive until tdfs_free_graph */

#define TDFS_GRAPH_VALIDATE 1u    /* check: offs monotone, offs[n] == nnz, lists strictly increasing,
                                      no self-loops, ids in range, symmetric -> TDFS_E_GRAPH_FORMAT */
#define TDFS_GRAPH_NORMALIZE 2u   /* HOST_COPY only: symmetrise, drop self-loops and duplicates, sort lists */
#define TDFS_GRAPH_DEGREE_ORDER 4u /* HOST_COPY only: the device graph renumbers vertices by (degree, id) rank, so the
                                      symmetry-breaking constraints f(a) < f(b) compare degree ranks (R35):
                                      counts are unchanged (any total order picks one embedding per copy); enumerated
                                      tuples are mapped back to the caller's ids (a representative per copy chosen by
                                      rank, not by id); shards and edge tasks follow the renumbered CSR order */

typedef struct {
  int64_t n;             /* number of vertices */
  int64_t nnz;           /* number of directed adjacency entries (= 2|E| for a valid graph) */
  const int64_t* offs;   /* [n+1]: N(v) = adj[offs[v] .. offs[v+1]) */
  const int32_t* adj;    /* [nnz]: neighbour ids, each list sorted ascending */
  const uint8_t* label;  /* [n] or NULL (unlabeled: every label is 0) */
  int32_t mem;           /* TDFS_MEM_HOST_COPY or TDFS_MEM_DEVICE_BORROW */
  uint32_t flags;        /* TDFS_GRAPH_VALIDATE | TDFS_GRAPH_NORMALIZE */
  int64_t hub_bitmap_bytes; /* device bytes for hub adjacency bitmaps (n bits per hub, vertices of degree
                               >= 256, highest degree first): 0 = default 256 MB, < 0 = none */
} tdfs_csr;

/* Load a CSR graph onto CUDA device `device`.  Uploads (HOST_COPY) or borrows the
 * arrays, computes d_max and the per-entry source array used by the edge tasks
 * (PAPER.md:120-122), builds the hub bitmaps.  Without VALIDATE the offsets and the
 * id range [0, n) are still checked (cheaply).  Errors: INVALID_ARG, GRAPH_FORMAT,
 * ID_RANGE, OOM, CUDA. */
int tdfs_load_graph(const tdfs_csr* g, int device, void* stream, tdfs_graph** out);

/* Load from an undirected edge list (host arrays, m pairs; any orientation,
 * duplicates and self-loops allowed -- they are normalised away on the host with
 * multiple threads).  label: host [n] or NULL. */
int tdfs_load_edges(int64_t n, int64_t m, const int32_t* src, const int32_t* dst, const uint8_t* label,
                    uint32_t flags /* 0 or TDFS_GRAPH_DEGREE_ORDER */, int64_t hub_bitmap_bytes /* as in tdfs_csr */,
                    int device, void* stream, tdfs_graph** out);

/* n, undirected edge count m = nnz/2, maximum degree, number of labels (max+1, 1 if unlabeled). */
int tdfs_graph_info(const tdfs_graph* g, int64_t* n, int64_t* m, int64_t* dmax, int32_t* nlabels);

/* Device pointers of the resident CSR (offs int64[n+1], adj int32[nnz], label uint8[n] or NULL). */
int tdfs_graph_device_arrays(const tdfs_graph* g, const int64_t** offs, const int32_t** adj,
                             const uint8_t** label);

void tdfs_free_graph(tdfs_graph* g);

/* ------------------------------------------------------------------ query plan
 * Host planner (PAPER.md:56, :75 matching order; :77 backward neighbours
 * B^pi(u_i); :29, :460 symmetry breaking from Aut(G_Q)).  Its cost is negligible
 * "as G_Q is small".
 */
typedef struct tdfs_plan tdfs_plan; /* opaque, library-owned, host-only */

typedef struct {
  const int32_t* order;        /* NULL = automatic greedy order; else a permutation of 0..k-1 whose every
                                  prefix is connected (order[1] adjacent to order[0]) */
  const int32_t* constraints;  /* pairs (a, b) meaning f(a) < f(b), 2*n_constraints ints */
  int32_t n_constraints;       /* -1 = automatic full symmetry breaking (stabilizer chain of Aut(Q)),
                                   0 = none (count every embedding), > 0 = use the given pairs */
} tdfs_plan_opts;

/* qedges: n_qedges pairs (0-based, duplicates ignored, no self-loops); qlabel: [k] in 0..255 or NULL
 * (NULL = unlabeled query: no label test).  opts NULL = {NULL, NULL, -1}.
 * Errors: INVALID_ARG, QUERY_TOO_LARGE, QUERY_DISCONNECTED, LABEL_RANGE. */
int tdfs_plan_query(int32_t k, int32_t n_qedges, const int32_t* qedges, const int32_t* qlabel,
                    const tdfs_plan_opts* opts, tdfs_plan** out);
int tdfs_plan_order(const tdfs_plan* p, int32_t* order /* [k] */);
int tdfs_plan_constraints(const tdfs_plan* p, int32_t* pairs /* [2*cap] */, int32_t cap, int32_t* n_out);
int tdfs_plan_aut_size(const tdfs_plan* p, int64_t* n_aut); /* |Aut(Q)| (label-preserving) */
int tdfs_plan_k(const tdfs_plan* p, int32_t* k);
void tdfs_free_plan(tdfs_plan* p);

/* ------------------------------------------------------------------ run
 * One kernel launch per job: persistent warps, each taking a
 * task from the lock-free queue Q_task (Alg. 3) before a new
 * chunk of initial edge tasks, depth-first backtracking
 * with timeout splitting (Alg. 4), paged stacks from a device
 * page pool (Alg. 5), Eq. (1) candidate generation by
 * warp-cooperative sorted-set intersection.
 */
#define TDFS_RUN_STATS 1u           /* fill tdfs_stats (slower kernel variant) */
#define TDFS_RUN_TRACE 2u           /* test hook: record enqueued tasks (see tdfs_test.h) */
#define TDFS_RUN_NO_REUSE 4u        /* ablation: disable set-intersection result reuse */
#define TDFS_RUN_NO_SHORTCUT 8u     /* ablation: always scan the last level (no count-only window shortcut) */
#define TDFS_RUN_NO_HUB_BITMAP 16u  /* ablation: probe hub adjacency lists by search, not by bitmap */
#define TDFS_RUN_NO_LEAF_STAGE 32u  /* ablation: no shared-memory staging of the last position's fixed part */
#define TDFS_RUN_ARRAY_STACKS 128u  /* ablation: array-based stack memory (d_max ids per warp-level up front, identity page tables: no page is ever allocated; Tables V-VIII) */
#define TDFS_RUN_NO_RANGE_TASKS 256u /* ablation: k = 4 timeout splits push one task per sibling instead of id-range tasks (R30) */

/* Partition of the initial edge tasks over shard_world ranks. */
#define TDFS_SHARD_ROUND_ROBIN 0      /* directed edge e (CSR index) -> rank e mod W */
#define TDFS_SHARD_DEGREE_BALANCED 1  /* heavy roots (cost = sum of neighbour degrees > total/(64 W)) dealt by
                                         edge round-robin; the other roots dealt whole in snake order of
                                         decreasing cost (R31) */
#define TDFS_SHARD_BLOCKED 2          /* blocks of 1024 consecutive directed edges dealt round-robin: block b ->
                                         rank b mod W (keeps a root's edges on one GPU; R36) */
#define TDFS_SHARD_BLOCK_EDGES 1024

typedef struct {
  int64_t tau_ns;              /* timeout tau; default 10 ms;
                                  < 0 = infinity ("No Steal"); 0 = split at every eligible step */
  int32_t chunk;               /* initial edge tasks per fetch; default 8; 1..32 */
  int64_t queue_ints;          /* Q_task capacity N in ints; default 3,000,000; N/3 tasks */
  int32_t page_bytes;          /* stack page size; default 8192; power of two >= 128 (:388) */
  int32_t page_table_entries;  /* per stack level; 0 = auto ceil(4*d_max/page_bytes) (paper fixes 40, :350) */
  int64_t pool_bytes;          /* page pool size; 0 = auto */
  int32_t blocks;              /* 0 = auto: SM count x resident blocks per SM (persistent) */
  int32_t warps_per_block;     /* 0 = auto (4) */
  int32_t shard_rank;          /* this GPU's share of the initial edge tasks (see shard_policy); */
  int32_t shard_world;         /*   1 = every directed edge */
  uint32_t flags;              /* TDFS_RUN_* */
  int32_t shard_policy;        /* TDFS_SHARD_ROUND_ROBIN (default) or TDFS_SHARD_DEGREE_BALANCED */
  int32_t reserved_;           /* 0 */
  uint64_t* shared_cursor;     /* NULL, or a device pointer (this device's memory or a peer's, e.g. from
                                  tdfs_shared_cursor_open) to a uint64 chunk cursor over ALL nnz directed edges,
                                  zeroed before the job and shared by every rank's concurrent job on the same
                                  graph (cross-GPU dynamic balancing; PAPER.md:122
                                  omits migration).  Overrides shard_rank/world/policy: each rank takes chunks
                                  from the shared cursor with system-scope atomics until it is exhausted. */
} tdfs_run_opts;

void tdfs_run_opts_default(tdfs_run_opts* o);

typedef struct {
  uint64_t nodes_per_level[TDFS_MAX_K + 1]; /* [p]: admissible partial matches of length p+1 (p >= 1) */
  uint64_t adj_bytes;         /* algorithmic bytes W: sum over extensions of
                                 4*|operand| + 16 per backward operand */
  uint64_t tasks_enqueued, tasks_dequeued, timeouts, queue_full;
  uint64_t pages_used;        /* pages taken from the pool (high-water, never freed) */
  uint64_t edges_scanned;     /* directed edges of this shard examined */
  uint64_t edges_filtered_in; /* of those, passing the edge filter */
  uint64_t chunks_fetched;
  float kernel_ms;            /* CUDA-event time of the matching kernel */
  int32_t grid_blocks, warps_per_block, page_table_entries, pad_;
  uint64_t pool_pages;
  uint64_t stream_bytes;      /* roofline bytes (R32): sum over extensions of 16 B per Eq. (1)
                                 operand + 4 B x |smallest constraint-windowed Eq. (1) source| (operands and
                                 reusable earlier candidate sets; 0 for a count-only last position) */
  uint64_t warp_exit_first_ns; /* load balance inside the GPU: when the first / an average / the last warp */
  uint64_t warp_exit_mean_ns;  /*   last found no work (queue empty, edges exhausted), from the kernel's first */
  uint64_t warp_exit_last_ns;  /*   warp start (ns); last - mean is the straggler tail that timeout
                                  splitting shortens */
} tdfs_stats;

/* Bytes of caller-owned device workspace needed for one job (256-byte aligned). */
size_t tdfs_workspace_bytes(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o);

/* Count |M(G, Q, C)| over this shard's initial tasks.
 *  workspace: device, >= tdfs_workspace_bytes, 256-byte aligned, exclusively used by this call
 *             until it completes on `stream`.
 *  d_count:   optional device uint64 receiving the count (TDFS_COUNT_INVALID on device failure).
 *  h_count:   optional host pointer; if non-NULL (or stats non-NULL) the call synchronises the
 *             stream and returns the device status; if NULL the call is asynchronous.
 *  stats:     optional; implies synchronous execution with the instrumented kernel variant.
 * Errors: INVALID_ARG, WORKSPACE, STACK_EXHAUSTED (no count written), CUDA. */
int tdfs_count(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
               size_t ws_bytes, void* stream, uint64_t* d_count, uint64_t* h_count, tdfs_stats* stats);

/* Enumerate M(G, Q, C) ("output S") over this shard.
 *  d_out: device int32[cap * k]; tuple i is d_out[i*k .. i*k+k), indexed by QUERY VERTEX id
 *         (not by matching-order position); tuples appear in no particular order.
 *  n_total: host; receives |M| (exact even on overflow).  Synchronous.
 * Errors: as tdfs_count, plus OUTPUT_OVERFLOW when |M| > cap (first cap tuples written). */
int tdfs_enumerate(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                   size_t ws_bytes, void* stream, int32_t* d_out, uint64_t cap, uint64_t* n_total,
                   tdfs_stats* stats);

/* Streaming enumerate ("output S"): every match of this shard,
 * without a capacity limit.  The kernel writes tuples (indexed by query vertex id, as in
 * tdfs_enumerate) into the caller-owned device ring d_ring[ring_cap * k] and waits for free space;
 * the calling thread drains it chunk by chunk (ring_cap / 8 tuples, copied to pinned host memory on
 * a side stream while the kernel runs) into sink(tuples, n, k, user) -- host memory valid during the
 * call only; a nonzero return stops delivery (the kernel still finishes and *n_total stays exact;
 * the call then returns TDFS_E_INVALID_ARG).  Synchronous.  ring_cap: positive multiple of 8.
 * Errors: as tdfs_count, plus INVALID_ARG. */
typedef int (*tdfs_tuple_sink)(const int32_t* tuples, uint64_t n, int32_t k, void* user);
int tdfs_enumerate_stream(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                          size_t ws_bytes, void* stream, int32_t* d_ring, uint64_t ring_cap, tdfs_tuple_sink sink,
                          void* user, uint64_t* n_total);
/* tdfs_enumerate_stream into a rank-local binary file: n_total rows of k little-endian int32
 * (query-vertex order), no header; tuples in no particular order. */
int tdfs_enumerate_to_file(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                           size_t ws_bytes, void* stream, int32_t* d_ring, uint64_t ring_cap, const char* path,
                           uint64_t* n_total);

/* Status of the last job run in `workspace` (device-side error word), synchronising `stream`. */
int tdfs_workspace_status(const void* workspace, void* stream);

/* ------------------------------------------------------------------ multi-GPU helpers
 * Owner rank of every directed edge under a shard policy (host only, no GPU needed):
 *  offs[n+1], adj[nnz] a CSR as in tdfs_csr (host); owner[nnz] receives the rank in [0, world) of the
 *  initial edge task e (the kernel's shard rank r processes exactly the edges with owner[e] == r).
 * Errors: INVALID_ARG (world < 1, unknown policy, NULL, nnz >= 2^31 for DEGREE_BALANCED). */
int tdfs_partition_edges(int64_t n, int64_t nnz, const int64_t* offs, const int32_t* adj, int32_t world,
                         int32_t policy, int32_t* owner);

/* A uint64 chunk cursor in this process's device memory that other processes (ranks on peer GPUs
 * of the same node, or on the same GPU) can map: *d_cursor is the local device pointer, ipc_handle
 * (64 bytes, cudaIpcMemHandle_t) is what the other ranks pass to tdfs_shared_cursor_open.  The
 * cursor is zeroed on `stream` by tdfs_shared_cursor_reset before each job. */
int tdfs_shared_cursor_create(int device, uint64_t** d_cursor, void* ipc_handle /* 64 bytes */);
int tdfs_shared_cursor_open(int device, const void* ipc_handle, uint64_t** d_cursor);
int tdfs_shared_cursor_reset(uint64_t* d_cursor, void* stream);
/* Close a cursor obtained from _open (opened = 1) or free one from _create (opened = 0). */
int tdfs_shared_cursor_close(uint64_t* d_cursor, int opened);

#ifdef __cplusplus
}
#endif
#endif /* TDFS_H_ */
