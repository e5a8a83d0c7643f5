// Device primitives shared by the matching kernel and the test hooks:
// PTX helpers, the lock-free task queue Q_task (Alg. 3) and the paged stack
// levels (Alg. 5).  Included inside `namespace tdfs { namespace { ... } }`.
#pragma once

constexpr unsigned FULL = 0xffffffffu;
constexpr uint32_t NULL_PAGE = 0xffffffffu;
constexpr int ERR_STACK = 1;

// ------------------------------------------------------------ PTX helpers
__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(unsigned* p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ long long ld_relaxed_s64(const unsigned long long* p) {
  long long v;
  asm volatile("ld.relaxed.gpu.global.s64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ long long ld_relaxed_sys_s64(const unsigned long long* p) {
  long long v;
  asm volatile("ld.relaxed.sys.global.s64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int ld_relaxed_s32(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int ld_relaxed_i32(const int32_t* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// L2 residency hints (north_star "Blackwell L2 residency hints for hub adjacency lists"): a
// cache policy built by createpolicy and attached to a read-only load with .L2::cache_hint.
// evict_last keeps the line in L2 ahead of normal lines; evict_first lets it go first.
__device__ __forceinline__ unsigned long long l2_evict_last() {
  unsigned long long p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long l2_evict_first() {
  unsigned long long p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned ldg_hint(const unsigned* a, unsigned long long pol) {
  unsigned v;
  asm("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(pol));
  return v;
}
__device__ __forceinline__ int ldg_hint(const int* a, unsigned long long pol) {
  int v;
  asm("ld.global.nc.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(pol));
  return v;
}
__device__ __forceinline__ int4 ldg_hint4(const int4* a, unsigned long long pol) {
  int4 v;
  asm("ld.global.nc.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
      : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(a), "l"(pol));
  return v;
}

__device__ __forceinline__ unsigned long long* ctr(const KParams& P, int i) { return P.ctr + i * kCounterStride; }

__device__ __forceinline__ int read_error(const KParams& P) {
  return ld_relaxed_s32(reinterpret_cast<const int*>(ctr(P, C_ERROR)));
}
__device__ __forceinline__ void raise_error(const KParams& P, int code) {
  atomicCAS(reinterpret_cast<unsigned long long*>(ctr(P, C_ERROR)), 0ull, (unsigned long long)code);
}

// lower_bound of v in B[0, n) (sorted), n < 2^31 (halving search).
__device__ __forceinline__ int lower_bound_dev(const int32_t* __restrict__ B, int n, int v) {
  int base = 0;
  while (n > 0) {
    const int half = n >> 1;
    if (__ldg(B + base + half) < v) {
      base += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return base;
}

// ------------------------------------------------------------ Q_task (Alg. 3)
// Bounded MPMC ring of 16-byte slots with 64-bit monotone tickets (R13).
// `free` / `avail` play the role of the paper's `size` (capacity check before the
// ticket); the per-slot sequence word replaces the three
// atomicCAS / atomicExch handshakes on the -1 sentinel.
struct Queue {
  QSlot* slots;
  uint64_t nslots;  // ring size, a power of two >= the capacity P.qcap (the `free` counter bounds occupancy)
  unsigned long long *head, *tail, *avail, *free_;
};

__device__ __forceinline__ Queue make_queue(const KParams& P) {
  return Queue{P.slots, P.qslots, ctr(P, C_QHEAD), ctr(P, C_QTAIL), ctr(P, C_QAVAIL), ctr(P, C_QFREE)};
}

// lane 0: reserve r consecutive tickets; returns ~0 if the queue is full (enqueue -> false).
__device__ __forceinline__ unsigned long long q_reserve(const Queue& q, int r) {
  long long old = (long long)atomicAdd(q.free_, (unsigned long long)(-(long long)r));
  if (old < r) {
    atomicAdd(q.free_, (unsigned long long)r);
    return ~0ull;
  }
  return atomicAdd(q.tail, (unsigned long long)r);
}

// A task in registers (see QSlot).
struct Task {
  int hdr;
  int v[6];
};

// one lane: write task into the slot of ticket t and publish it
__device__ __forceinline__ void q_publish(const Queue& q, unsigned long long t, const Task& k) {
  QSlot* s = q.slots + (t & (q.nslots - 1));
  unsigned want = (unsigned)t;
  while (ld_acquire_u32(&s->seq) != want) __nanosleep(32);
  volatile QSlot* vs = s;
  vs->hdr = k.hdr;
#pragma unroll
  for (int i = 0; i < 6; i++) vs->v[i] = k.v[i];
  st_release_u32(&s->seq, (unsigned)(t + 1));
}

// lane 0: Alg. 3 dequeue.  Returns false when empty.
__device__ __forceinline__ bool q_pop(const Queue& q, Task& k) {
  if (ld_relaxed_s64(q.avail) <= 0) return false;
  long long old = (long long)atomicAdd(q.avail, (unsigned long long)(-1ll));
  if (old <= 0) {
    atomicAdd(q.avail, 1ull);
    return false;
  }
  unsigned long long h = atomicAdd(q.head, 1ull);
  QSlot* s = q.slots + (h & (q.nslots - 1));
  unsigned want = (unsigned)(h + 1);
  while (ld_acquire_u32(&s->seq) != want) __nanosleep(32);
  volatile QSlot* vs = s;
  k.hdr = vs->hdr;
#pragma unroll
  for (int i = 0; i < 6; i++) k.v[i] = vs->v[i];
  st_release_u32(&s->seq, (unsigned)(h + q.nslots));
  atomicAdd(q.free_, 1ull);
  return true;
}

// Warp-cooperative push of the tasks held by the lanes in `mask` (lane i pushes its own task).
// Returns false if the queue is full (nothing pushed).  The test trace records (v1, v2, v3) of
// edge tasks as <v1, v2, -2> and of 3-prefix tasks as <v1, v2, v3>; range tasks as <v1, v2, -3 - d>.
__device__ __forceinline__ bool q_push_warp(const KParams& P, const Queue& q, unsigned mask, const Task& k, int lane) {
  int r = __popc(mask);
  if (r == 0) return true;
  unsigned long long t = 0;
  if (lane == 0) t = q_reserve(q, r);
  t = __shfl_sync(FULL, t, 0);
  if (t == ~0ull) return false;
  if (mask >> lane & 1u) {
    unsigned long long my = t + __popc(mask & lanemask_lt());
    q_publish(q, my, k);
  }
  __syncwarp();
  if (P.trace) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(ctr(P, C_TRACE), (unsigned long long)r);
    base = __shfl_sync(FULL, base, 0);
    if (mask >> lane & 1u) {
      unsigned long long i = base + __popc(mask & lanemask_lt());
      if ((long long)i < P.trace_cap) {
        const int kind = k.hdr & 15;
        P.trace[3 * i] = k.v[0];
        P.trace[3 * i + 1] = k.v[1];
        P.trace[3 * i + 2] = kind == TASK_EDGE ? -2 : kind == TASK_PREFIX ? k.v[2] : -3 - (k.hdr >> 4);
      }
    }
  }
  if (lane == 0) {
    __threadfence();
    atomicAdd(q.avail, (unsigned long long)r);
  }
  __syncwarp();
  return true;
}

// ------------------------------------------------------------ paged stacks (Alg. 5)
struct PagedLevel {
  uint32_t* table;  // E entries
};

__device__ __forceinline__ int32_t* page_base(const KParams& P, uint32_t pg) {
  return P.pool + ((size_t)pg << P.page_shift);
}

// lane 0: make sure table[p] exists; returns page id or NULL_PAGE on exhaustion
__device__ __forceinline__ uint32_t ensure_page(const KParams& P, uint32_t* table, int p) {
  if (p >= P.E) return NULL_PAGE;
  uint32_t pg = table[p];
  if (pg == NULL_PAGE) {
    unsigned long long id = atomicAdd(ctr(P, C_POOL), 1ull);
    if (id >= P.n_pages) return NULL_PAGE;
    pg = (uint32_t)id;
    table[p] = pg;
  }
  return pg;
}

// Paged reader (the [] operator of Alg. 5 for reads): element pos of a level.
__device__ __forceinline__ int32_t paged_read(const KParams& P, const uint32_t* table, long long pos) {
  uint32_t pg = table[pos >> P.page_shift];
  return page_base(P, pg)[pos & ((1ll << P.page_shift) - 1)];
}

// Warp-level paged writer state for one extension (sequential batches).
struct PagedWriter {
  uint32_t* table;
  int cur_p;        // page index currently cached
  uint32_t cur_pg;  // its page id
};

// Write the lanes in `ballot` (ballot-compacted) at positions
// pos0 .. pos0 + popc - 1.  Returns false on stack exhaustion.
__device__ __forceinline__ bool paged_write(const KParams& P, PagedWriter& w, unsigned ballot, long long pos0,
                                            int v, int lane) {
  int cnt = __popc(ballot);
  if (cnt == 0) return true;
  const int shift = P.page_shift;
  int pf = (int)(pos0 >> shift);
  int pl = (int)((pos0 + cnt - 1) >> shift);
  uint32_t pgf = w.cur_pg, pgl = w.cur_pg;
  if (pf != w.cur_p || pl != w.cur_p) {
    uint32_t a = 0, b = 0;
    if (lane == 0) {
      a = ensure_page(P, w.table, pf);
      b = (pl == pf) ? a : ensure_page(P, w.table, pl);
    }
    a = __shfl_sync(FULL, a, 0);
    b = __shfl_sync(FULL, b, 0);
    if (a == NULL_PAGE || b == NULL_PAGE) return false;
    pgf = a;
    pgl = b;
    w.cur_p = pl;
    w.cur_pg = b;
  }
  if (ballot >> lane & 1u) {
    long long pos = pos0 + __popc(ballot & lanemask_lt());
    uint32_t pg = ((int)(pos >> shift) == pf) ? pgf : pgl;
    page_base(P, pg)[pos & ((1ll << shift) - 1)] = v;
  }
  return true;
}

