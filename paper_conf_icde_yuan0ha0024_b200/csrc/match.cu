// The T-DFS hot path on sm_100a: one persistent kernel per job.
//
// Per warp (the basic processing unit):
//   outer loop   take a task from Q_task first (Alg. 4 l.1-3), else the
//                next chunk of initial edge tasks of this GPU's shard (l.4-5,
//                PAPER.md:122), edge-filtered in the warp; exit when
//                no work remains anywhere (termination rule, R12).
//   DFS          iterative backtracking over matching-order positions with per-level
//                size/iter (Alg. 2 / Alg. 4); S, size[],
//                iter[] live in lane-indexed registers (lane p holds position p).
//   timeout      before descending at a split-eligible level (task prefix <= 3
//                matched vertices) lane 0 reads %globaltimer; when
//                now - t0 >= tau the current and all remaining siblings are pushed to
//                Q_task and the warp backtracks (Alg. 4 l.12-21);
//                a full queue resets t0 (l.18-20).
//   stacks       each stored level is a page table over fixed-size pages taken from a
//                device pool on first touch and kept for the whole job (Alg. 5,
//                PAPER.md:340-390); a batch of <= 32 outputs crosses <= 1 page
//                boundary; allocation is warp-uniform (lane 0), so no
//                divergent leader election is needed.  Exhaustion is an error, never a
//                truncated count.
//   Eq. (1)      candidates = intersection of the backward neighbours' sorted
//                adjacency lists, computed warp-cooperatively: the
//                shortest operand is streamed with coalesced loads, one element per
//                lane, and each other operand is probed by per-lane binary search
//                whose lower bound advances batch by batch;
//                symmetry-breaking constraints become a [lo, hi) id window applied by
//                binary search before the scan; injectivity,
//                label and degree filters are fused; survivors are
//                compacted with __ballot_sync/__popc into the next level, or only
//                counted at the last level.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <climits>
#include <thread>
#include <cstdlib>
#include <cstring>

#include "internal.h"

namespace tdfs {
namespace {

#include "prims.cuh"

// per-leaf entry of a flat leaf batch (shared memory, one per lane of the batch)
struct __align__(16) LeafMeta {
  long long b0;  // N(x) = adj[b0, b0 + deg)
  int deg;
  int hid;       // hub bitmap row of x, -1 = none
  int lo, hi;    // stream B: F window of this leaf F[lo, hi); stream A: N(x)[lo, hi), the entries inside
                 // [F_min, F_max] (the range its probes search)
  int s, e;      // streamed element range: stream A F-coordinates [s, e) of the 16-byte aligned F,
                 // stream B N(x) entries [b0 + s, b0 + e) (narrowed to [F_min, F_max])
};
// 32 entries + 33 prefix ints (padded to 16 B) + a 128-id transpose buffer
constexpr int kMetaBytesPerWarp = 32 * (int)sizeof(LeafMeta) + 144 + 512;
__host__ __device__ inline size_t smem_meta_offset(int wpb, int fcap) {
  return ((size_t)wpb * fcap * sizeof(int) + 15) & ~(size_t)15;
}
__host__ __device__ inline size_t smem_bytes(int wpb, int fcap) {
  return smem_meta_offset(wpb, fcap) + (size_t)wpb * kMetaBytesPerWarp;
}

extern __shared__ __align__(16) int tdfs_smem[];  // [F stages of the block's warps][batch entries of the warps]

// ------------------------------------------------------------ warp context
template <bool STATS>
struct Ctx {
  int lane;
  int sreg;                 // lane p: S[p]
  int lsize, liter;         // lane p: size[p], iter[p] (a level holds <= d_max < 2^31 ids)
  unsigned long long count;  // warp-uniform
  unsigned long long t0;     // lane 0: task start time
  unsigned long long lnodes; // lane p: nodes[p]   (STATS)
  unsigned long long wbytes, sbytes, enq, deq, touts, qfull, scanned, edges_in, chunks;  // lane 0 (STATS)
  uint32_t* tables;         // this warp's page tables [n_levels][E]
  int* sF;                  // this warp's shared-memory stage for the leaf set F (P.fcap ints)
  int wlev;                 // range task: level d whose candidates are restricted to ids in [wlo, whi); 0 = none
  int wlo, whi;
  int wmode;                // 1: level wlev built as the slice only; 2: built whole, iterated in the slice
  int wend;                 // mode 2: iteration end index at level wlev (INT_MAX otherwise)
  int own;                  // lowest stored level whose FULL candidate list this warp built for the current
                            // prefix (2 for edge tasks, 3 for 3-prefix tasks, wlev / wlev+1 for range tasks):
                            // only lists at levels >= own may be reused (set-intersection reuse)
};

__device__ __forceinline__ int getS(int sreg, int p) { return __shfl_sync(FULL, sreg, p); }

// timeout test (lane 0 decides, broadcast)
template <bool STATS>
__device__ __forceinline__ bool timed_out(const KParams& P, Ctx<STATS>& c) {
  if (P.tau_ns < 0) return false;
  int t = 0;
  if (c.lane == 0) t = (long long)(globaltimer() - c.t0) >= P.tau_ns;
  return __shfl_sync(FULL, t, 0) != 0;
}

// lower_bound of v in the paged list [lo, hi) of a stored level
__device__ __forceinline__ long long paged_lower_bound(const KParams& P, const uint32_t* table, long long lo,
                                                       long long hi, int v) {
  while (lo < hi) {
    long long mid = (lo + hi) >> 1;
    if (paged_read(P, table, mid) < v) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// Warp-cooperative lower_bound of v in the sorted global list L[0, n): each round the 32
// lanes sample the remaining range at 32 evenly spaced points (one load per lane) and keep
// one stride, so a list of n ids takes ceil(log32 n) dependent loads instead of log2 n.
__device__ __forceinline__ long long warp_lower_bound(const int32_t* __restrict__ L, long long n, int v, int lane) {
  long long lo = 0;
  while (n > 32) {
    const long long step = (n + 31) >> 5;
    const long long i = lo + (long long)(lane + 1) * step - 1;  // last id of stride `lane`
    const bool less = i < lo + n && __ldg(L + i) < v;
    const int c = __popc(__ballot_sync(FULL, less));             // strides entirely below v
    lo += (long long)c * step;
    n = min(step, n - (long long)c * step);
  }
  const bool less = lane < n && __ldg(L + lo + lane) < v;
  return lo + __popc(__ballot_sync(FULL, less));
}

// Warp-cooperative lower_bound of v in the paged list [lo, hi) of a stored level (same
// scheme as warp_lower_bound; each sample is a page-table load and a page load).
__device__ __forceinline__ long long warp_paged_lower_bound(const KParams& P, const uint32_t* table, long long lo,
                                                            long long hi, int v, int lane) {
  long long n = hi - lo;
  while (n > 32) {
    const long long step = (n + 31) >> 5;
    const long long i = lo + (long long)(lane + 1) * step - 1;
    const bool less = i < lo + n && paged_read(P, table, i) < v;
    const int c = __popc(__ballot_sync(FULL, less));
    lo += (long long)c * step;
    n = min(step, n - (long long)c * step);
  }
  const bool less = lane < n && paged_read(P, table, lo + lane) < v;
  return lo + __popc(__ballot_sync(FULL, less));
}

// Enumerate output of match number idx, t[p] = f(pi_p) (written indexed by query vertex id).
// Capacity mode (P.ring_chunk == 0): out[idx] if idx < cap, else dropped (the total stays exact).
// Streaming mode (NEXT-2): out is a ring of cap tuples in ring_chunk-tuple chunks drained by the
// host (tdfs_enumerate_stream); the lane waits until its slot is free (idx < consumed + cap), writes
// the tuple, and counts it into its chunk's fill word; the host copies a chunk out once it is full.
// A lane only waits for its own slot, so the chunk the host waits for always completes.
__device__ __forceinline__ void emit_tuple(const KParams& P, unsigned long long idx, const int* t, int k) {
  if (P.ring_chunk == 0) {
    if (idx < P.cap)
      for (int p = 0; p < k; p++) P.out[idx * k + P.plan.order[p]] = P.orig ? __ldg(P.orig + t[p]) : t[p];
    return;
  }
  const unsigned long long* consumed = ctr(P, C_CONSUMED);
  while (idx >= (unsigned long long)ld_relaxed_s64(consumed) + P.cap) __nanosleep(2000);
  const unsigned long long slot = idx % P.cap;
  for (int p = 0; p < k; p++) P.out[slot * k + P.plan.order[p]] = P.orig ? __ldg(P.orig + t[p]) : t[p];
  __threadfence();
  atomicAdd(P.ring_fill + (idx / P.ring_chunk) % P.ring_nchunks, 1ull);
}

// STATS only (roofline bytes R32): |C(r) within [lo, hi)| from the definition, for a stored
// position r whose list this warp did not build (a <v1,v2,v3> or range task): the ids of the
// intersection of r's backward lists inside r's window and [lo, hi) that pass r's injectivity,
// label and degree tests.  Streams r's first operand, binary-searches the others.
template <bool STATS>
__device__ long long source_size_def(const KParams& P, Ctx<STATS>& c, int r, int lo, int hi) {
  const DevPlan& pl = P.plan;
  const int lane = c.lane;
  lo = max(lo, (int)__reduce_max_sync(FULL, ((pl.lo_mask[r] >> lane) & 1u) ? (unsigned)(c.sreg + 1) : 0u));
  hi = min(hi, (int)__reduce_min_sync(FULL, ((pl.hi_mask[r] >> lane) & 1u) ? (unsigned)c.sreg : (unsigned)INT_MAX));
  if (lo >= hi) return 0;
  const uint32_t bm = pl.bwd[r];
  const int x0 = getS(c.sreg, __ffs(bm) - 1);
  const long long b0 = __ldg(P.offs + x0), e0 = __ldg(P.offs + x0 + 1);
  const long long s = b0 + warp_lower_bound(P.adj + b0, e0 - b0, lo, lane);
  long long total = 0;
  for (long long base = s; base < e0; base += 32) {
    const long long i = base + lane;
    const int v = i < e0 ? __ldg(P.adj + i) : INT_MAX;
    bool ok = i < e0 && v < hi;
    for (uint32_t m = bm & (bm - 1); m; m &= m - 1) {
      const int x = getS(c.sreg, __ffs(m) - 1);
      if (ok) {
        const long long b = __ldg(P.offs + x), e = __ldg(P.offs + x + 1);
        const int pos = lower_bound_dev(P.adj + b, (int)(e - b), v);
        ok = pos < e - b && __ldg(P.adj + b + pos) == v;
      }
    }
    for (uint32_t m = pl.inj_mask[r]; m; m &= m - 1) {
      const int sj = getS(c.sreg, __ffs(m) - 1);
      ok = ok && v != sj;
    }
    if (ok && pl.label[r] >= 0) ok = (P.label ? (int)__ldg(P.label + v) : 0) == pl.label[r];
    if (ok && pl.deg_min[r] > 0) ok = (__ldg(P.offs + v + 1) - __ldg(P.offs + v)) >= pl.deg_min[r];
    total += __popc(__ballot_sync(FULL, ok));
    if (!__any_sync(FULL, i < e0 && v < hi)) break;
  }
  return total;
}

// Candidate generation for position d (Eq. 1 + fused filters).
// MODE_OUT: 0 = store into the paged level of d; 1 = count only (last position);
//           2 = enumerate (last position); 3 = stage into shared memory (d = kVF, the
//           S[k-2]-independent part of the last position), or return -2 without
//           writing when the streamed operand exceeds the stage (P.fcap ids).
// Set-intersection reuse starts only from lists this warp built in full (levels >= c.own).
// Returns the number of candidates, or -1 on stack exhaustion.
template <int MODE_OUT, bool STATS>
__device__ long long extend(const KParams& P, Ctx<STATS>& c, int d) {
  const int lane = c.lane;
  const DevPlan& pl = P.plan;
  int r = pl.reuse[d];
  if (r >= 0 && r < c.own) r = -1;
  const uint32_t bm_all = pl.bwd[d];
  // set-intersection result reuse: start from C(r), intersect the rest
  const uint32_t bm = (r >= 0) ? (bm_all & ~pl.bwd[r]) : bm_all;
  const int nops = __popc(bm);
  // global operand t (lane t < nops) = adjacency list of S[j_t], j_t = t-th set bit of bm
  int jt = 0;
  {
    uint32_t m = bm;
    for (int i = 0; i < lane && m; i++) m &= m - 1;
    jt = m ? (__ffs(m) - 1) : 0;
  }
  const int sj = __shfl_sync(FULL, c.sreg, jt);
  long long ob = 0, oe = 0;
  int hid = -1;
  if (lane < nops) {
    ob = __ldg(P.offs + sj);
    oe = __ldg(P.offs + sj + 1);
    if (P.hub_id) hid = __ldg(P.hub_id + sj);
  }
  // a range task re-extends part of a level-2 list its splitter already counted (STATS only)
  const bool counted = STATS && MODE_OUT != 3 && d != c.wlev;
  if (counted) {  // W of SURVEY 8(d) counts every backward operand of Eq. (1), reused or not
    const bool mine = (bm_all >> lane) & 1u;
    unsigned long long wb = 0;
    if (mine) wb = (unsigned long long)(4 * (__ldg(P.offs + c.sreg + 1) - __ldg(P.offs + c.sreg)) + 16);
    for (int o = 16; o > 0; o >>= 1) wb += __shfl_xor_sync(FULL, wb, o);
    if (lane == 0) c.wbytes += wb;
  }
  // constraint window [lo, hi)
  const uint32_t lom = pl.lo_mask[d], him = pl.hi_mask[d];
  int lo = __reduce_max_sync(FULL, (lom >> lane & 1u) ? c.sreg + 1 : 0);
  int hi = (int)__reduce_min_sync(FULL, (him >> lane & 1u) ? (unsigned)c.sreg : (unsigned)INT_MAX);
  if (d == c.wlev && c.wmode == 1) {  // range task: only the level-d candidates in [wlo, whi)
    lo = max(lo, c.wlo);
    hi = min(hi, c.whi);
  }
  if (counted) {  // roofline bytes R32: 16 B per operand + 4 B x the smallest windowed Eq. (1) source
    const bool mine = (bm_all >> lane) & 1u;
    unsigned wlen = UINT_MAX;
    if (mine && lo < hi) {
      const long long b = __ldg(P.offs + c.sreg), e = __ldg(P.offs + c.sreg + 1);
      const int n = (int)(e - b);
      const int a = lo > 0 ? lower_bound_dev(P.adj + b, n, lo) : 0;
      const int z = hi < INT_MAX ? a + lower_bound_dev(P.adj + b + a, n - a, hi) : n;
      wlen = (unsigned)(z - a);
    }
    unsigned mn = __reduce_min_sync(FULL, wlen);
    if (lo < hi)
      for (uint32_t sm = pl.src_mask[d]; sm; sm &= sm - 1) {  // stored candidate sets C(r) (reuse sources)
        const int rr = __ffs(sm) - 1;
        long long len;
        if (rr < c.own) {
          len = source_size_def(P, c, rr, lo, hi);  // list not built (in full) by this warp: from the definition
        } else {
          const uint32_t* tb = c.tables + (size_t)(rr - 2) * P.E;
          const long long rs = __shfl_sync(FULL, c.lsize, rr);
          const long long a = lo > 0 ? warp_paged_lower_bound(P, tb, 0, rs, lo, lane) : 0;
          len = (hi < INT_MAX ? warp_paged_lower_bound(P, tb, a, rs, hi, lane) : rs) - a;
        }
        mn = min(mn, (unsigned)len);
      }
    const int nall = __popc(bm_all);
    if (lane == 0) c.sbytes += 16ull * nall + ((lo >= hi || pl.cnt_only[d] || mn == UINT_MAX) ? 0ull : 4ull * mn);
  }
  if (lo >= hi) return 0;
  const bool windowed = (lo > 0 || hi < INT_MAX);
  if (windowed) {
    // warp-cooperative window search, one operand at a time (ceil(log32 n) dependent loads)
    for (int t = 0; t < nops; t++) {
      const long long tb = __shfl_sync(FULL, ob, t), te = __shfl_sync(FULL, oe, t);
      const long long a = lo > 0 ? warp_lower_bound(P.adj + tb, te - tb, lo, lane) : 0;
      const long long b = hi < INT_MAX ? a + warp_lower_bound(P.adj + tb + a, te - tb - a, hi, lane) : te - tb;
      if (lane == t) { ob = tb + a; oe = tb + b; }
    }
  }
  // the reused list, windowed
  const uint32_t* rtable = nullptr;
  long long ra = 0, rb = 0;
  if (r >= 0) {
    rtable = c.tables + (size_t)(r - 2) * P.E;
    const long long rsize = __shfl_sync(FULL, c.lsize, r);
    // when the window includes v > S[r]: C(r) is sorted and S[r] = C(r)[iter[r] - 1], so the
    // window starts at or after iter[r] -- exactly there when lo = S[r] + 1 (no search)
    long long r0 = 0;
    bool ra_known = false;
    if ((lom >> r) & 1u) {
      r0 = __shfl_sync(FULL, c.liter, r);
      ra_known = (lo == getS(c.sreg, r) + 1);
    }
    if (ra_known) ra = r0;
    else ra = lo > 0 ? warp_paged_lower_bound(P, rtable, r0, rsize, lo, lane) : 0;
    rb = hi < INT_MAX ? warp_paged_lower_bound(P, rtable, ra, rsize, hi, lane) : rsize;
    if (ra >= rb) return 0;
  }
  const uint32_t injm = pl.inj_mask[d];

  // count-only last position with a single remaining list and no per-element filter:
  // |C(d)| = |window| - |matched vertices inside it| (no scan)
  if (MODE_OUT == 1 && (pl.shortcut[d] & (r >= 0 ? 1u : 2u)) && (r >= 0 || nops == 1)) {
    const long long b0 = __shfl_sync(FULL, ob, 0), e0 = __shfl_sync(FULL, oe, 0);
    const long long len = (r >= 0) ? (rb - ra) : (e0 - b0);
    bool hit = false;
    if ((injm >> lane) & 1u) {
      const int s = c.sreg;
      if (s >= lo && s < hi && len > 0) {
        if (r >= 0) {
          const long long i = paged_lower_bound(P, rtable, ra, rb, s);
          hit = i < rb && paged_read(P, rtable, i) == s;
        } else {
          const int i = lower_bound_dev(P.adj + b0, (int)len, s);
          hit = i < len && __ldg(P.adj + b0 + i) == s;
        }
      }
    }
    const long long total = len - __popc(__ballot_sync(FULL, hit));
    if (counted && d < kVF && lane == d) c.lnodes += (unsigned long long)total;
    return total;
  }

  // the streamed operand A: the reused list, else the shortest windowed adjacency list
  int tA = -1;
  long long bA, eA;
  if (r >= 0) {
    bA = ra;
    eA = rb;
  } else {
    const long long len = (lane < nops) ? (oe - ob) : LLONG_MAX;
    const unsigned minlen = __reduce_min_sync(FULL, (unsigned)min(len, (long long)UINT_MAX));
    if (minlen == 0) return 0;
    tA = __ffs(__ballot_sync(FULL, lane < nops && (unsigned)len == minlen)) - 1;
    bA = __shfl_sync(FULL, ob, tA);
    eA = __shfl_sync(FULL, oe, tA);
  }
  if (r >= 0 && nops > 0) {
    const unsigned z = __ballot_sync(FULL, lane < nops && oe <= ob);
    if (z) return 0;
  }
  if (MODE_OUT == 3 && eA - bA > (long long)P.fcap) return -2;
  const uint32_t others = __ballot_sync(FULL, lane < nops && lane != tA);
  const int need_label = (r >= 0 && pl.label[r] == pl.label[d]) ? -1 : pl.label[d];
  const int dmin = (r >= 0 && pl.deg_min[r] >= pl.deg_min[d]) ? 0 : pl.deg_min[d];

  PagedWriter w;
  w.table = c.tables + (size_t)(d - 2) * P.E;
  w.cur_p = -1;
  w.cur_pg = NULL_PAGE;
  long long total = 0;

  for (long long base = bA; base < eA; base += 32) {
    const long long i = base + lane;
    const bool inr = i < eA;
    int v = INT_MAX;
    if (inr) v = (r >= 0) ? paged_read(P, rtable, i) : __ldg(P.adj + i);
    bool ok = inr;
    const int last_lane = (int)min(31ll, eA - 1 - base);
    // probe the other operands: merge (32-id register chunks, shuffle search) when the
    // operand is at most kMergeRatio times longer than A, else per-lane binary search;
    // either way the operand's lower bound advances batch by batch
    uint32_t om = others;
    while (om) {
      const int t = __ffs(om) - 1;
      om &= om - 1;
      const long long tb = __shfl_sync(FULL, ob, t);
      const long long te = __shfl_sync(FULL, oe, t);
      const int th = __shfl_sync(FULL, hid, t);
      if (th >= 0) {
        // hub operand: one bitmap load per candidate (v is inside the window already)
        if (ok) ok = (__ldg(P.hub_bits + (long long)th * P.hub_words + (v >> 5)) >> (v & 31)) & 1u;
      } else if ((te - tb) <= (long long)kMergeRatio * (eA - base)) {
        // warp merge: walk B in coalesced 32-id chunks until a chunk reaches the batch max
        const int amax = __shfl_sync(FULL, v, last_lane);
        bool found = false;
        long long ptr = tb;
        while (ptr < te) {
          const long long j = ptr + lane;
          const int bv = (j < te) ? __ldg(P.adj + j) : INT_MAX;
          int pos = 0;
#pragma unroll
          for (int s = 16; s > 0; s >>= 1)
            if (__shfl_sync(FULL, bv, pos + s - 1) < v) pos += s;
          found |= (__shfl_sync(FULL, bv, pos) == v);
          const int bmax = __shfl_sync(FULL, bv, 31);
          if (bmax >= amax) break;
          ptr += 32;
        }
        ok = ok && found;
        if (lane == t) ob = min(ptr, te);
      } else {
        int pos = (int)(te - tb);
        const bool probe = inr && (ok || lane == last_lane);
        if (probe) pos = lower_bound_dev(P.adj + tb, (int)(te - tb), v);
        if (ok) ok = (pos < te - tb) && __ldg(P.adj + tb + pos) == v;
        const int adv = __shfl_sync(FULL, pos, last_lane);
        if (lane == t) ob = tb + adv;
      }
      if (!__any_sync(FULL, ok)) break;
    }
    // fused filters: injectivity, label, degree
    if (injm) {
      uint32_t m = injm;
      while (m) {
        const int j = __ffs(m) - 1;
        m &= m - 1;
        const int s = getS(c.sreg, j);
        ok = ok && (v != s);
      }
    }
    if (need_label >= 0 && ok) ok = (P.label ? (int)__ldg(P.label + v) : 0) == need_label;
    if (dmin > 0 && ok) ok = (__ldg(P.offs + v + 1) - __ldg(P.offs + v)) >= dmin;
    const unsigned bal = __ballot_sync(FULL, ok);
    const int cnt = __popc(bal);
    if (MODE_OUT == 0) {
      if (!paged_write(P, w, bal, total, v, lane)) return -1;
    } else if (MODE_OUT == 3) {
      if (ok) c.sF[total + __popc(bal & lanemask_lt())] = v;
    } else if (MODE_OUT == 2 && cnt) {
      unsigned long long ob0 = 0;
      if (lane == 0) ob0 = atomicAdd(ctr(P, C_OUTCUR), (unsigned long long)cnt);
      ob0 = __shfl_sync(FULL, ob0, 0);
      const int k = pl.k;
      const unsigned long long idx = ob0 + __popc(bal & lanemask_lt());
      int t[kMaxK];
#pragma unroll
      for (int p = 0; p < kMaxK - 1; p++) t[p] = getS(c.sreg, p);
      t[k - 1] = v;
      if (ok) emit_tuple(P, idx, t, k);
    }
    total += cnt;
  }
  if (MODE_OUT == 3) __syncwarp();
  if (counted && d < kVF && lane == d) c.lnodes += (unsigned long long)total;
  return total;
}

// Per-vertex probe metadata of N(x): CSR range, hub bitmap row.
struct VMeta {
  long long b0, b1;  // N(x) = adj[b0, b1)
  int hid;           // hub bitmap row, -1 = none
};

__device__ __forceinline__ VMeta load_vmeta(const KParams& P, int x) {
  VMeta m;
  m.b0 = __ldg(P.offs + x);
  m.b1 = __ldg(P.offs + x + 1);
  m.hid = P.hub_id ? __ldg(P.hub_id + x) : -1;
  return m;
}

// The staged leaf set F of a level-(k-2) list: either materialised in this warp's shared
// memory (sorted, every S[k-2]-independent filter applied), or -- when F is a window of a
// single adjacency list N(y) with no per-element filter (lf_byref) and y has a hub bitmap --
// referenced in place: F = adj[offs[y] + a, offs[y] + b) and "w in F" is "w in [F_min, F_max]
// and w in N(y)" by y's bitmap (no copy, no size cap).
struct FRef {
  const int* F;  // sorted ids F[0, nF) (shared or global memory)
  int hid;       // by reference: y's bitmap row; -1 = F is materialised in shared memory
  unsigned fix;  // by reference, plans without an N(S[k-2]) operand: lanes j whose S[j] must differ from
                 // the leaf's candidates (injectivity at positions <= k-3) and lies inside F
};

// matched vertices S[j] (j in fr.fix) inside F[lo, hi): subtracted from a !lf_var leaf count
// (warp-collective: every lane calls it, with its own window)
__device__ __forceinline__ int fixed_in_window(const FRef& fr, int sreg, int lo, int hi) {
  int n = 0;
  const bool nonempty = lo < hi;
  const int fmin = nonempty ? fr.F[lo] : 1, fmax = nonempty ? fr.F[hi - 1] : 0;
  for (unsigned m = fr.fix; m; m &= m - 1) {
    const int s = __shfl_sync(FULL, sreg, __ffs(m) - 1);
    n += (s >= fmin && s <= fmax) ? 1 : 0;
  }
  return n;
}

// per-lane lower_bound of v in the sorted F[lo, hi) (shared or global memory)
__device__ __forceinline__ int lane_lower_bound(const int* F, int lo, int hi, int v) {
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (F[mid] < v) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

__device__ __forceinline__ int warp_excl_scan(int v, int lane) {
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  return x - v;
}

// Branch-free lower_bound of four values in the same sorted list L[lo, lo + n) (global, shared
// or generic memory): every step issues the four probes together (independent loads in flight)
// and all four share the trip count ceil(log2 n).  Results in r0..r3 (indices into L).
__device__ __forceinline__ void lower_bound4(const int* L, int lo, int n, int v0, int v1, int v2, int v3, int& r0,
                                             int& r1, int& r2, int& r3) {
  r0 = r1 = r2 = r3 = lo;
  if (n <= 0) return;
  while (n > 1) {
    const int half = n >> 1;
    const int a0 = L[r0 + half], a1 = L[r1 + half], a2 = L[r2 + half], a3 = L[r3 + half];
    r0 = a0 < v0 ? r0 + half : r0;
    r1 = a1 < v1 ? r1 + half : r1;
    r2 = a2 < v2 ? r2 + half : r2;
    r3 = a3 < v3 ? r3 + half : r3;
    n -= half;
  }
  r0 += L[r0] < v0;
  r1 += L[r1] < v1;
  r2 += L[r2] < v2;
  r3 += L[r3] < v3;
}

// L2 residency hints (north_star; prims.cuh ldg_hint), a build-time experiment, off by default: measured
// with no gain.  Bit 0: hub-bitmap probes evict_last; bit 1: stream-B N(x) loads
// evict_first; bit 2 (with bit 1): N(x) of a hub leaf evict_last instead.
#ifndef TDFS_L2HINT
#define TDFS_L2HINT 0
#endif
__device__ __forceinline__ unsigned bit_of(const uint32_t* row, int v) {
#if TDFS_L2HINT & 1
  return (ldg_hint(row + (v >> 5), l2_evict_last()) >> (v & 31)) & 1u;
#else
  return (__ldg(row + (v >> 5)) >> (v & 31)) & 1u;
#endif
}

// A whole batch of nb <= 32 staged leaves at once: lane j
// holds leaf x_j = S[k-2] and N(x_j)'s metadata.  The count is only summed, so the batch's
// work is flattened into two load-balanced streams over the leaves' elements:
//   A: leaves where streaming F is cheaper: elements F[lo_j .. hi_j), each probed in N(x_j)
//      (hub bitmap, else binary search);
//   B: the others: elements of N(x_j) narrowed to [F_min_j, F_max_j], each probed in F (y's
//      bitmap when F is referenced, else a shared-memory binary search).
// Both streams are walked in aligned 16-byte groups: one 128-bit load gives a lane four
// consecutive ids of one leaf (north_star "vectorised coalesced 128-bit adjacency loads"),
// whose four probes are then issued together.  A lane moves to the next leaf by walking the
// batch's prefix sums in shared memory; hits are summed per lane and reduced once per batch.
template <bool STATS>
__device__ long long leaf_batch(const KParams& P, Ctx<STATS>& c, const FRef& fr, int nF, int nb, int x,
                                const VMeta& m) {
  const DevPlan& pl = P.plan;
  const int lane = c.lane;
  const int* F = fr.F;
  const bool byref = fr.hid >= 0;
  const bool act = lane < nb;
  int lo = 0, hi = nF;
  if (act && pl.lf_lo_var) lo = lane_lower_bound(F, 0, nF, x + 1);
  if (act && pl.lf_hi_var) hi = lane_lower_bound(F, lo, nF, x);
  if (!pl.lf_var) {
    const int nfix = fr.fix ? fixed_in_window(fr, c.sreg, act ? lo : 0, act ? hi : 0) : 0;
    long long cnt = (act && lo < hi) ? hi - lo - nfix : 0;
    if (cnt && pl.lf_inj_var) {  // x itself inside F[lo, hi)?
      if (fr.hid >= 0) {            // referenced F of a hub y: range test + one bitmap load
        cnt -= (x >= F[lo] && x <= F[hi - 1] &&
                bit_of(P.hub_bits + (long long)fr.hid * P.hub_words, x)) ? 1 : 0;
      } else {
        const int i = lane_lower_bound(F, lo, hi, x);
        cnt -= (i < hi && F[i] == x) ? 1 : 0;
      }
    }
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(FULL, cnt, o);
    __syncwarp();  // every lane's reads of F are done before the next list overwrites it
    return cnt;
  }
  // F is walked from its 16-byte aligned base: F = Fal + fo
  const int fo = (int)((reinterpret_cast<uintptr_t>(F) >> 2) & 3u);
  const int* const Fal = F - fo;
  const int a = (act && lo < hi) ? hi - lo : 0;
  int bs = 0, be = act ? (int)(m.b1 - m.b0) : 0;
  int gA = 0, gB = 0;  // this leaf's 16-byte groups in stream A / B
  if (a > 0 && be > 0) {
    // N(x) narrowed to [F_min, F_max] (both bounds by search for long lists)
    if (be >= 64) {
      const int* N = P.adj + m.b0;
      bs = lower_bound_dev(N, be, F[lo]);
      be = bs + lower_bound_dev(N + bs, be - bs, F[hi - 1] + 1);
    }
    const int b = be - bs;
    if (b > 0) {
      const int lgb = 32 - __clz(be), lga = 32 - __clz(a);
      const long long uA = m.hid >= 0 ? kUaHub : 3 + lgb;
      const long long uB = byref ? kUbRef : 3 + (lga >> 1);
      if ((long long)a * uA <= (long long)b * uB) gA = ((fo + hi + 3) >> 2) - ((fo + lo) >> 2);
      else gB = (int)(((m.b0 + be + 3) >> 2) - ((m.b0 + bs) >> 2));
    }
  }
  char* const wbase = reinterpret_cast<char*>(tdfs_smem) + P.meta_off + (int)(threadIdx.x >> 5) * kMetaBytesPerWarp;
  LeafMeta* meta = reinterpret_cast<LeafMeta*>(wbase);
  int* pre = reinterpret_cast<int*>(wbase + 32 * sizeof(LeafMeta));
  // 128-id transpose buffer: a lane loads 4 consecutive ids with one 128-bit load, but the probes
  // of ids 4L..4L+3 by lane L would hit 4 sectors per lane; after the transpose lane L probes ids
  // L, L+32, L+64, L+96 of the warp's 128, so adjacent lanes probe adjacent sorted ids (shared
  // bitmap words / sectors) -- measured 17.9 sectors per warp load request before
  int* const tb = reinterpret_cast<int*>(wbase + 32 * sizeof(LeafMeta) + 144);
  if (act) {
    LeafMeta e;
    e.b0 = m.b0;
    e.deg = (int)(m.b1 - m.b0);
    e.hid = m.hid;
    e.lo = gA ? bs : lo;  // A: the narrowed N(x) range [bs, be) searched; B: the F window
    e.hi = gA ? be : hi;
    e.s = gA ? fo + lo : bs;
    e.e = gA ? fo + hi : be;
    meta[lane] = e;
  }
  unsigned cnt = 0;
  // stream A: F elements of leaf j probed in N(x_j)
  {
    const int p = warp_excl_scan(gA, lane);
    const int tot = __shfl_sync(FULL, p + gA, 31);
    __syncwarp();
    pre[lane] = act ? p : tot;
    if (lane == 0) pre[32] = tot;
    __syncwarp();
    int j = -1, jn = 0, pj = 0, g0 = 0, sj = 0, ej = 0, hidj = -1, degj = 0, pb = 0;
    long long b0j = 0;
    for (int base = 0; base < tot; base += 32) {
      const int idx = base + lane;
      int4 q = make_int4(-1, -1, -1, -1);
      bool k0 = false, k1 = false, k2 = false, k3 = false;
      if (idx < tot) {
        if (idx >= jn) {  // move to the leaf holding idx (per lane, shared-memory reads)
          do { ++j; jn = pre[j + 1]; } while (jn <= idx);
          pj = pre[j];
          const LeafMeta e = meta[j];
          sj = e.s; ej = e.e; hidj = e.hid; b0j = e.b0;
          pb = e.lo;  // N(x_j)[lo, hi) holds every id in [F_min_j, F_max_j]
          degj = e.hi;
          g0 = sj >> 2;
        }
        const int g = g0 + idx - pj;
        q = *reinterpret_cast<const int4*>(Fal + 4 * g);
        const int i0 = 4 * g;
        k0 = i0 >= sj && i0 < ej;
        k1 = i0 + 1 >= sj && i0 + 1 < ej;
        k2 = i0 + 2 >= sj && i0 + 2 < ej;
        k3 = i0 + 3 >= sj && i0 + 3 < ej;
      }
      // hub leaves: transposed bitmap probes (the row of id L + 32t is its loader lane's: (L >> 2) + 8t)
      const bool hub = idx < tot && hidj >= 0;
      if (__any_sync(FULL, hub)) {
        reinterpret_cast<int4*>(tb)[lane] =
            make_int4(hub && k0 ? q.x : -1, hub && k1 ? q.y : -1, hub && k2 ? q.z : -1, hub && k3 ? q.w : -1);
        __syncwarp();
#pragma unroll
        for (int t = 0; t < 4; t++) {
          const int w = tb[lane + 32 * t];
          const int row = __shfl_sync(FULL, hidj, (lane >> 2) + 8 * t);
          if (w >= 0) cnt += bit_of(P.hub_bits + (long long)row * P.hub_words, w);
        }
        __syncwarp();
      }
      if (idx < tot && hidj < 0) {
        {
          // this lane's ids of one leaf increase group by group: search N(x_j) from the last hit;
          // ids outside the leaf's window search as +inf (they sit past every valid id)
          const int v0 = k0 ? q.x : INT_MAX, v1 = k1 ? q.y : INT_MAX, v2 = k2 ? q.z : INT_MAX, v3 = k3 ? q.w : INT_MAX;
          const int* N = P.adj + b0j;
          int r0, r1, r2, r3;
          lower_bound4(N, pb, degj - pb, v0, v1, v2, v3, r0, r1, r2, r3);
          cnt += (k0 && r0 < degj && N[r0] == v0) + (k1 && r1 < degj && N[r1] == v1) +
                 (k2 && r2 < degj && N[r2] == v2) + (k3 && r3 < degj && N[r3] == v3);
          pb = k0 ? r0 : pb;
          pb = k1 ? r1 : pb;
          pb = k2 ? r2 : pb;
          pb = k3 ? r3 : pb;
        }
      }
    }
  }
  // stream B: N(x_j) elements inside [F_min_j, F_max_j] probed in F
  {
    const int p = warp_excl_scan(gB, lane);
    const int tot = __shfl_sync(FULL, p + gB, 31);
    __syncwarp();
    pre[lane] = act ? p : tot;
    if (lane == 0) pre[32] = tot;
    __syncwarp();
    const int4* const adj4 = reinterpret_cast<const int4*>(P.adj);
    const uint32_t* const frow = fr.hid >= 0 ? P.hub_bits + (long long)fr.hid * P.hub_words : nullptr;
    int j = -1, jn = 0, pj = 0, loj = 0, hij = 0, fminj = 0, fmaxj = 0;
#if TDFS_L2HINT & 4
    int hidB = -1;
#endif
    long long g0 = 0, sj = 0, ej = 0;
    for (int base = 0; base < tot; base += 32) {
      const int idx = base + lane;
      int4 q = make_int4(-1, -1, -1, -1);
      bool k0 = false, k1 = false, k2 = false, k3 = false;
      if (idx < tot) {
        if (idx >= jn) {
          do { ++j; jn = pre[j + 1]; } while (jn <= idx);
          pj = pre[j];
          const LeafMeta e = meta[j];
          loj = e.lo; hij = e.hi;
#if TDFS_L2HINT & 4
          hidB = e.hid;
#endif
          sj = e.b0 + e.s;
          ej = e.b0 + e.e;
          g0 = sj >> 2;
          fminj = F[loj];
          fmaxj = F[hij - 1];
        }
        const long long g = g0 + idx - pj;
#if TDFS_L2HINT & 2
#if TDFS_L2HINT & 4
        q = ldg_hint4(adj4 + g, hidB >= 0 ? l2_evict_last() : l2_evict_first());
#else
        q = ldg_hint4(adj4 + g, l2_evict_first());
#endif
#else
        q = __ldg(adj4 + g);
#endif
        const long long i0 = g << 2;
        k0 = i0 >= sj && i0 < ej && q.x >= fminj && q.x <= fmaxj;
        k1 = i0 + 1 >= sj && i0 + 1 < ej && q.y >= fminj && q.y <= fmaxj;
        k2 = i0 + 2 >= sj && i0 + 2 < ej && q.z >= fminj && q.z <= fmaxj;
        k3 = i0 + 3 >= sj && i0 + 3 < ej && q.w >= fminj && q.w <= fmaxj;
      }
      if (frow) {  // warp-uniform: transposed probes of y's bitmap
        reinterpret_cast<int4*>(tb)[lane] = make_int4(k0 ? q.x : -1, k1 ? q.y : -1, k2 ? q.z : -1, k3 ? q.w : -1);
        __syncwarp();
#pragma unroll
        for (int t = 0; t < 4; t++) {
          const int w = tb[lane + 32 * t];
          if (w >= 0) cnt += bit_of(frow, w);
        }
        __syncwarp();
      } else if (idx < tot) {
        {
          // F in shared memory: four lockstep searches; a kept id is <= F_max so its index is < hi
          int r0, r1, r2, r3;
          lower_bound4(F, loj, hij - loj, q.x, q.y, q.z, q.w, r0, r1, r2, r3);
          cnt += (k0 && F[r0] == q.x) + (k1 && F[r1] == q.y) + (k2 && F[r2] == q.z) + (k3 && F[r3] == q.w);
        }
      }
    }
  }
  __syncwarp();
  return (long long)__reduce_add_sync(FULL, cnt);
}
// Stage F for the level-(k-2) list just built (see FRef).  Returns |F|, or -2 when F
// would have to be materialised and exceeds the shared-memory stage (generic per leaf).
template <bool STATS>
__device__ int stage_leaf_set(const KParams& P, Ctx<STATS>& c, FRef& fr) {
  const DevPlan& pl = P.plan;
  const int lane = c.lane;
  __syncwarp();  // the previous list's leaves are done reading the stage before it is overwritten
  fr.F = c.sF;
  fr.hid = -1;
  fr.fix = 0;
  if (pl.lf_byref) {
    const int y = getS(c.sreg, __ffs(pl.bwd[kVF]) - 1);
    const VMeta my = load_vmeta(P, y);
    if (my.hid >= 0) {
      const uint32_t lom = pl.lo_mask[kVF], him = pl.hi_mask[kVF];
      const int wlo = __reduce_max_sync(FULL, (lom >> lane & 1u) ? c.sreg + 1 : 0);
      const int whi = (int)__reduce_min_sync(FULL, (him >> lane & 1u) ? (unsigned)c.sreg : (unsigned)INT_MAX);
      if (wlo >= whi) return 0;
      const long long n = my.b1 - my.b0;
      const long long a = wlo > 0 ? warp_lower_bound(P.adj + my.b0, n, wlo, lane) : 0;
      const long long b = whi < INT_MAX ? a + warp_lower_bound(P.adj + my.b0 + a, n - a, whi, lane) : n;
      fr.F = P.adj + my.b0 + a;
      fr.hid = my.hid;
      if (const uint32_t im = pl.inj_mask[kVF]) {  // matched S[j] (j <= k-3) that lie inside F
        bool in = false;
        if ((im >> lane) & 1u) {
          const int s = c.sreg;
          if (s >= wlo && s < whi) in = bit_of(P.hub_bits + (long long)my.hid * P.hub_words, s);
        }
        fr.fix = __ballot_sync(FULL, in);
      }
      return (int)(b - a);
    }
  }
  return (int)extend<3, STATS>(P, c, kVF);
}

// Push <S0, S1, L[2][i]> for i in [from, size) -- timeout split of level 2, one 3-prefix task
// per remaining sibling.  Returns the first index NOT pushed (size on success).
template <bool STATS>
__device__ long long split_level2(const KParams& P, Ctx<STATS>& c, const Queue& q, long long from, long long size) {
  const uint32_t* table = c.tables;  // level index 0 = position 2
  Task k;
  k.hdr = TASK_PREFIX;
  k.v[0] = getS(c.sreg, 0);
  k.v[1] = getS(c.sreg, 1);
  k.v[3] = k.v[4] = k.v[5] = -1;
  for (long long base = from; base < size; base += 32) {
    const long long i = base + c.lane;
    k.v[2] = 0;
    if (i < size) k.v[2] = paged_read(P, table, i);
    const unsigned mask = __ballot_sync(FULL, i < size);
    if (!q_push_warp(P, q, mask, k, c.lane)) {
      if (STATS && c.lane == 0) c.qfull++;
      return base;
    }
    if (STATS && c.lane == 0) c.enq += __popc(mask);
  }
  return size;
}

// Timeout split of level d (2 <= d <= kMaxRangeLevel) into range tasks (R30/R33): instead
// of one task per remaining sibling, push at most 32 tasks <S0 .. S_{d-1}, lo, hi>, each covering
// >= 32 consecutive siblings C[i .. i+g) by id range [C[i], C[i+g]) (the last one up to this list's
// own bound).  A receiver rebuilds that slice of level d (one more window bound), or the whole list
// when a later position reuses it, and continues the DFS below it; it can time out and split its
// slice again.  Returns false if the queue is full.
template <bool STATS>
__device__ bool split_ranges(const KParams& P, Ctx<STATS>& c, const Queue& q, int d, int from, int size) {
  const int lane = c.lane;
  const uint32_t* table = c.tables + (size_t)(d - 2) * P.E;
  const int rem = size - from;
  const int g = max(kRangeMin, (rem + kRangeMaxT - 1) / kRangeMaxT);
  const int ntask = (rem + g - 1) / g;
  const int i0 = from + lane * g, i1 = i0 + g;
  Task k;
  k.hdr = TASK_RANGE | (d << 4);
#pragma unroll
  for (int i = 0; i < 6; i++) k.v[i] = getS(c.sreg, i);  // lanes >= d overwritten / unused
  int lo = 0, hi = (c.wlev == d) ? c.whi : INT_MAX;
  if (lane < ntask) lo = paged_read(P, table, i0);
  if (lane < ntask && i1 < size) hi = paged_read(P, table, i1);
#pragma unroll
  for (int i = 2; i <= kMaxRangeLevel; i++)
    if (i == d) { k.v[i] = lo; k.v[i + 1] = hi; }
  const unsigned mask = ntask >= 32 ? FULL : ((1u << ntask) - 1u);
  if (!q_push_warp(P, q, mask, k, lane)) {
    if (STATS && lane == 0) c.qfull++;
    return false;
  }
  if (STATS && lane == 0) c.enq += ntask;
  return true;
}

// Depth-first search below a prefix S[0..start-1] (Alg. 4 l.7-28).
// Returns false on error.
template <int MODE, bool STATS>
__device__ bool dfs(const KParams& P, Ctx<STATS>& c, const Queue& q, int start) {
  const int k = P.plan.k;
  const int lane = c.lane;
  if (start == k - 1) {
    long long n = (MODE == 1) ? extend<2, STATS>(P, c, start) : extend<1, STATS>(P, c, start);
    c.count += (unsigned long long)n;
    return true;
  }
  // leaf staging (count jobs): F of the virtual position kVF, once per level-(k-2) list
  const bool use_lf = MODE == 0 && !STATS && P.plan.lf_on && P.fcap > 0;
  int nF = -1;  // staged |F|, -1 = not staged (generic Eq. (1) per leaf)
  FRef fr;
  int d = start;
  long long sz = extend<0, STATS>(P, c, d);
  if (sz < 0) return false;
  if (lane == d) { c.lsize = (int)sz; c.liter = 0; }
  if (start == c.wlev && c.wmode == 2) {  // range task over a whole list: iterate [wlo, whi) only
    const uint32_t* tb = c.tables + (size_t)(d - 2) * P.E;
    const long long ib = warp_paged_lower_bound(P, tb, 0, sz, c.wlo, lane);
    const long long ie = c.whi < INT_MAX ? warp_paged_lower_bound(P, tb, ib, sz, c.whi, lane) : sz;
    if (lane == d) c.liter = (int)ib;
    c.wend = (int)ie;
  }
  if (use_lf && d == k - 2) {
    nF = sz >= 2 ? stage_leaf_set(P, c, fr) : -1;
    if (nF == 0 && lane == d) c.liter = (int)sz;  // F empty: no leaf below this list
  }
  int glev = 0;  // after a full queue at level glev: descend once in place before re-checking (progress at tau = 0)
  for (;;) {
    const int it = __shfl_sync(FULL, c.liter, d);
    const int size = d == c.wlev ? min(__shfl_sync(FULL, c.lsize, d), c.wend) : __shfl_sync(FULL, c.lsize, d);
    if (it < size) {
      if (((P.split_mask >> d) & 1u) && d != glev && timed_out(P, c)) {
        // timeout: push the current and all remaining siblings, then backtrack
        if (STATS && lane == 0) c.touts++;
        if ((P.range_mask >> d) & 1u) {
          // <= kRangeMin remaining siblings finish in place (tasks strictly shrink: progress at tau = 0)
          if (size - it <= kRangeMin) {
            if (lane == 0) c.t0 = globaltimer();
            glev = d;
            continue;
          }
          if (split_ranges(P, c, q, d, it, size)) {
            if (lane == d) c.liter = size;
            continue;
          }
          if (lane == 0) c.t0 = globaltimer();  // queue full: continue in place
          glev = d;
          continue;
        }
        long long upto = split_level2(P, c, q, it, size);  // d == 2: the paper's per-sibling tasks
        if (upto >= size) {
          if (lane == d) c.liter = size;
          continue;
        }
        // queue full: the pushed prefix is gone, continue in place with t0 reset
        if (lane == d) c.liter = (int)upto;
        if (lane == 0) c.t0 = globaltimer();
        glev = d;
        continue;
      }
      if (glev == d) glev = 0;
      const uint32_t* table = c.tables + (size_t)(d - 2) * P.E;
      if (d + 1 == k - 1 && use_lf && nF >= 0) {
        // staged leaves in batches of 32: the ids and N(x) metadata of the batch are
        // loaded by one lane each (independent loads), then each leaf is one |F ∩ N(x)|
        const int nb = min(32, size - it);
        const int vl = lane < nb ? paged_read(P, table, it + lane) : 0;
        VMeta ml = {0, 0, -1};
        if (lane < nb) ml = load_vmeta(P, vl);
        c.count += (unsigned long long)leaf_batch(P, c, fr, nF, nb, vl, ml);
        if (lane == d) c.liter = it + nb;
        continue;
      }
      const int v = paged_read(P, table, it);
      if (lane == d) { c.sreg = v; c.liter = it + 1; }
      if (d + 1 == k - 1) {
        long long n = (MODE == 1) ? extend<2, STATS>(P, c, d + 1) : extend<1, STATS>(P, c, d + 1);
        c.count += (unsigned long long)n;
      } else {
        d++;
        sz = extend<0, STATS>(P, c, d);
        if (sz < 0) return false;
        if (lane == d) { c.lsize = (int)sz; c.liter = 0; }
        if (use_lf && d == k - 2) {
          nF = sz >= 2 ? stage_leaf_set(P, c, fr) : -1;
          if (nF == 0 && lane == d) c.liter = (int)sz;
        }
      }
    } else {
      if (d == start) break;
      d--;
    }
  }
  return true;
}

// Process one chunk [j0, j1) of this shard's directed edges (Alg. 4 l.5, edge
// filtering PAPER.md:400).  Returns false on error.
template <int MODE, bool STATS>
__device__ bool run_chunk(const KParams& P, Ctx<STATS>& c, const Queue& q, long long j0, long long j1) {
  const int lane = c.lane;
  const DevPlan& pl = P.plan;
  const int k = pl.k;
  for (long long jb = j0; jb < j1; jb += 32) {
    const long long j = jb + lane;
    const bool inr = j < j1;
    int v0 = 0, v1 = 0;
    bool ok = inr;
    if (inr) {
      long long e;
      if (P.task_edges) {
        e = (long long)__ldg(P.task_edges + j);
      } else if (P.shard_block) {  // j-th edge of this rank's blocks: block ordinal j / B -> global block
        const long long ob = j / P.shard_block;
        e = (ob * P.shard_world + P.shard_rank) * P.shard_block + (j - ob * P.shard_block);
      } else {
        e = (long long)P.shard_rank + j * (long long)P.shard_world;
      }
      v0 = __ldg(P.src + e);
      v1 = __ldg(P.adj + e);
      if (pl.edge_cons == 1) ok = v0 < v1;
      else if (pl.edge_cons == -1) ok = v1 < v0;
      else if (pl.edge_cons == 2) ok = false;
      if (ok && pl.label[0] >= 0) ok = (P.label ? (int)__ldg(P.label + v0) : 0) == pl.label[0];
      if (ok && pl.label[1] >= 0) ok = (P.label ? (int)__ldg(P.label + v1) : 0) == pl.label[1];
      if (ok && pl.deg_min[0] > 1) ok = (__ldg(P.offs + v0 + 1) - __ldg(P.offs + v0)) >= pl.deg_min[0];
      if (ok && pl.deg_min[1] > 1) ok = (__ldg(P.offs + v1 + 1) - __ldg(P.offs + v1)) >= pl.deg_min[1];
    }
    unsigned mask = __ballot_sync(FULL, ok);
    if (STATS) {
      const unsigned scanned = __ballot_sync(FULL, inr);
      if (lane == 1) c.lnodes += __popc(mask);
      if (lane == 0) {
        c.scanned += __popc(scanned);
        c.edges_in += __popc(mask);
      }
    }
    if (k == 2) {  // the query is one edge: every filtered edge is a match
      const int cnt = __popc(mask);
      if (MODE == 1 && cnt) {
        unsigned long long ob0 = 0;
        if (lane == 0) ob0 = atomicAdd(ctr(P, C_OUTCUR), (unsigned long long)cnt);
        ob0 = __shfl_sync(FULL, ob0, 0);
        const unsigned long long idx = ob0 + __popc(mask & lanemask_lt());
        int t[kMaxK];
        t[0] = v0;
        t[1] = v1;
        if (ok) emit_tuple(P, idx, t, 2);
      }
      c.count += (unsigned long long)cnt;
      continue;
    }
    while (mask) {
      // timeout check before descending into the next edge (edge level is split-eligible)
      if (timed_out(P, c)) {
        if (STATS && lane == 0) c.touts++;
        Task et;
        et.hdr = TASK_EDGE;
        et.v[0] = v0;
        et.v[1] = v1;
        et.v[2] = -2;
        et.v[3] = et.v[4] = et.v[5] = -1;
        if (q_push_warp(P, q, mask, et, lane)) {
          if (STATS && lane == 0) c.enq += __popc(mask);
          mask = 0;
          break;
        }
        if (STATS && lane == 0) c.qfull++;
        if (lane == 0) c.t0 = globaltimer();
      }
      const int l = __ffs(mask) - 1;
      mask &= mask - 1;
      const int a = __shfl_sync(FULL, v0, l), b = __shfl_sync(FULL, v1, l);
      if (lane == 0) c.sreg = a;
      if (lane == 1) c.sreg = b;
      if (!dfs<MODE, STATS>(P, c, q, 2)) return false;
    }
    if (read_error(P)) return false;
  }
  return true;
}

// The persistent matching kernel.  MODE 0 = count, 1 = enumerate.
template <int MODE, bool STATS>
#ifndef TDFS_MIN_BLOCKS
#define TDFS_MIN_BLOCKS 12  // 40 registers: measured best of 8..16 on config 2
#endif
__global__ void __launch_bounds__(kBlockThreads, TDFS_MIN_BLOCKS) tdfs_kernel(const KParams P) {
  const int lane = threadIdx.x & 31;
  const long long gwarp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  Ctx<STATS> c;
  c.lane = lane;
  c.sreg = -1;
  c.lsize = 0;
  c.liter = 0;
  c.count = 0;
  c.t0 = 0;
  c.lnodes = 0;
  c.wbytes = c.sbytes = c.enq = c.deq = c.touts = c.qfull = c.scanned = c.edges_in = c.chunks = 0;
  c.wlev = 0;
  c.wlo = 0;
  c.whi = INT_MAX;
  c.wmode = 0;
  c.wend = INT_MAX;
  c.own = 2;
  c.tables = P.page_tables + (size_t)gwarp * (size_t)max(P.n_levels, 1) * (size_t)P.E;
  c.sF = tdfs_smem + (threadIdx.x >> 5) * P.fcap;
  const Queue q = make_queue(P);
  int* active = reinterpret_cast<int*>(ctr(P, C_ACTIVE));
  unsigned long long* cursor = P.gcursor;

  if (lane == 0) atomicAdd(active, 1);
  const unsigned long long t_start = STATS ? globaltimer() : 0ull;
  unsigned long long t_idle = t_start;
  if (STATS && P.stats && lane == 0) atomicMin(P.stats + S_T_START, t_start);
  bool busy = true;
  for (;;) {
    if (read_error(P)) break;
    if (!busy) {
      // idle: wait for queued tasks; exit when no warp is busy and the queue is empty
      int go = 0;
      if (lane == 0) {
        if (ld_relaxed_s64(q.avail) > 0) {
          atomicAdd(active, 1);
          go = 1;
        } else {
          __threadfence();
          go = (ld_relaxed_s32(active) == 0) ? -1 : 0;
        }
      }
      go = __shfl_sync(FULL, go, 0);
      if (go < 0) break;
      if (go == 0) {
        __nanosleep(256);
        continue;
      }
      busy = true;
    }
    // 1. Q_task first
    int got = 0;
    Task tk;
    if (lane == 0) {
      got = q_pop(q, tk);
      if (got) c.t0 = globaltimer();
    }
    got = __shfl_sync(FULL, got, 0);
    if (got) {
      const int hdr = __shfl_sync(FULL, tk.hdr, 0);
      int mine = 0;
#pragma unroll
      for (int i = 0; i < 6; i++) {
        const int x = __shfl_sync(FULL, tk.v[i], 0);
        if (lane == i) mine = x;
      }
      if (STATS && lane == 0) c.deq++;
      const int kind = hdr & 15, lev = hdr >> 4;
      int start = 2;
      if (kind == TASK_EDGE) {
        if (lane < 2) c.sreg = mine;
      } else if (kind == TASK_PREFIX) {
        if (lane < 3) c.sreg = mine;
        start = 3;
        c.own = 3;
      } else {  // TASK_RANGE at level lev: prefix S[0 .. lev-1], ids [lo, hi)
        if (lane < lev) c.sreg = mine;
        c.wlev = lev;
        c.wlo = __shfl_sync(FULL, mine, lev);
        c.whi = __shfl_sync(FULL, mine, lev + 1);
        c.wmode = ((P.reused_mask >> lev) & 1u) ? 2 : 1;
        c.own = c.wmode == 2 ? lev : lev + 1;
        start = lev;
      }
      const bool ok = dfs<MODE, STATS>(P, c, q, start);
      c.wlev = 0;
      c.wlo = 0;
      c.whi = INT_MAX;
      c.wmode = 0;
      c.wend = INT_MAX;
      c.own = 2;
      if (!ok) {
        raise_error(P, ERR_STACK);
        break;
      }
      continue;
    }
    // 2. next chunk of initial edge tasks
    long long j0 = P.n_tasks;
    if (lane == 0) {
      if (P.gshared) {  // cursor shared with other ranks / GPUs (NEXT-3): system-scope atomics
        if (ld_relaxed_sys_s64(cursor) < P.n_tasks) {
          j0 = (long long)atomicAdd_system(cursor, (unsigned long long)P.chunk);
          c.t0 = globaltimer();
        }
      } else if ((long long)ld_relaxed_s64(cursor) < P.n_tasks) {
        j0 = (long long)atomicAdd(cursor, (unsigned long long)P.chunk);
        c.t0 = globaltimer();
      }
    }
    j0 = __shfl_sync(FULL, j0, 0);
    if (j0 < P.n_tasks) {
      if (STATS && lane == 0) c.chunks++;
      long long j1 = min(j0 + (long long)P.chunk, (long long)P.n_tasks);
      if (!run_chunk<MODE, STATS>(P, c, q, j0, j1)) {
        raise_error(P, ERR_STACK);
        break;
      }
      continue;
    }
    // 3. nothing to do: become idle
    if (lane == 0) {
      __threadfence();
      atomicSub(active, 1);
      if (STATS) t_idle = globaltimer();  // the last of these is when this warp's work ended
    }
    busy = false;
  }
  if (busy && lane == 0) atomicSub(active, 1);
  // publish this warp's results
  if (lane == 0 && c.count) atomicAdd(ctr(P, C_COUNT), c.count);
  if (STATS && P.stats) {
    if (lane < kMaxK + 1 && c.lnodes) atomicAdd(P.stats + S_NODES + lane, c.lnodes);
    if (lane == 0) {
      atomicAdd(P.stats + S_ADJ_BYTES, c.wbytes);
      atomicAdd(P.stats + S_STREAM, c.sbytes);
      atomicAdd(P.stats + S_ENQ, c.enq);
      atomicAdd(P.stats + S_DEQ, c.deq);
      atomicAdd(P.stats + S_TIMEOUTS, c.touts);
      atomicAdd(P.stats + S_QFULL, c.qfull);
      atomicAdd(P.stats + S_EDGES_SCANNED, c.scanned);
      atomicAdd(P.stats + S_EDGES_IN, c.edges_in);
      atomicAdd(P.stats + S_CHUNKS, c.chunks);
      const unsigned long long te = t_idle;  // load balance: when this warp last ran out of work
      atomicMin(P.stats + S_T_EXIT_MIN, te);
      atomicMax(P.stats + S_T_EXIT_MAX, te);
      atomicAdd(P.stats + S_T_EXIT_SUM, te - t_start);
      atomicAdd(P.stats + S_WARPS, 1ull);
    }
  }
}

// Initialise the queue's per-slot sequence words for ticket base `base`.
__global__ void init_queue_kernel(QSlot* slots, unsigned long long cap, unsigned long long base) {
  for (unsigned long long s = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; s < cap;
       s += (unsigned long long)gridDim.x * blockDim.x) {
    unsigned long long first = base + ((s + cap - (base % cap)) % cap);  // first ticket >= base hitting slot s
    slots[s].seq = (unsigned)first;
    slots[s].hdr = -1;
    for (int i = 0; i < 6; i++) slots[s].v[i] = -1;
  }
}

__global__ void iota_u32_kernel(uint32_t* a, unsigned long long n) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    a[i] = (uint32_t)i;
}

__global__ void init_counters_kernel(unsigned long long* ctrs, unsigned long long qcap, unsigned long long base) {
  int i = threadIdx.x;
  if (i < C_NUM * kCounterStride) ctrs[i] = 0;
  __syncthreads();
  if (i == 0) {
    ctrs[C_QHEAD * kCounterStride] = base;
    ctrs[C_QTAIL * kCounterStride] = base;
    ctrs[C_QFREE * kCounterStride] = qcap;
  }
}

__global__ void finalize_kernel(const unsigned long long* ctrs, unsigned long long* d_count) {
  if (threadIdx.x == 0 && blockIdx.x == 0)
    *d_count = ctrs[C_ERROR * kCounterStride] ? TDFS_COUNT_INVALID : ctrs[C_COUNT * kCounterStride];
}

using KernelFn = void (*)(const KParams);
KernelFn pick_kernel(int mode, bool stats) {
  if (mode == 0) return stats ? tdfs_kernel<0, true> : tdfs_kernel<0, false>;
  return stats ? tdfs_kernel<1, true> : tdfs_kernel<1, false>;
}

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

int cuda_fail(cudaError_t e, const char* what) {
  return fail(TDFS_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

}  // namespace

// ------------------------------------------------------------------ host side
int blocks_per_sm(int device, int wpb, bool stats, bool enumerate, int fcap, int* out) {
  (void)device;
  int nb = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, pick_kernel(enumerate ? 1 : 0, stats), wpb * 32,
                                                                smem_bytes(wpb, fcap));
  if (e != cudaSuccess) return cuda_fail(e, "occupancy");
  if (nb < 1) return fail(TDFS_E_INVALID_ARG, "occupancy: the kernel cannot be resident with this block shape");
  *out = nb;
  return TDFS_OK;
}

int resolve_layout(const Graph* g, const Plan* p, const tdfs_run_opts* o, WsLayout* L) {
  if (!g || !p || !o || !L) return fail(TDFS_E_INVALID_ARG, "layout: NULL");
  if (o->chunk < 1 || o->chunk > 4096) return fail(TDFS_E_INVALID_ARG, "opts.chunk must be in [1, 4096]");
  if (o->queue_ints < 3) return fail(TDFS_E_INVALID_ARG, "opts.queue_ints must be >= 3");
  if (o->page_bytes < 128 || (o->page_bytes & (o->page_bytes - 1)))
    return fail(TDFS_E_INVALID_ARG, "opts.page_bytes must be a power of two >= 128");
  if (o->shard_world < 1 || o->shard_rank < 0 || o->shard_rank >= o->shard_world)
    return fail(TDFS_E_INVALID_ARG, "opts.shard_rank/shard_world");
  if (o->warps_per_block < 0 || o->blocks < 0 || o->page_table_entries < 0 || o->pool_bytes < 0)
    return fail(TDFS_E_INVALID_ARG, "opts: negative size");
  int dev = g->device;
  int sms = 0;
  cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) return cuda_fail(e, "device attribute");
  L->wpb = o->warps_per_block > 0 ? o->warps_per_block : 4;
  if (L->wpb > kBlockThreads / 32)  // the kernel's __launch_bounds__
    return fail(TDFS_E_INVALID_ARG, "opts.warps_per_block must be <= " + std::to_string(kBlockThreads / 32));
  if (o->shard_policy != TDFS_SHARD_ROUND_ROBIN && o->shard_policy != TDFS_SHARD_DEGREE_BALANCED &&
      o->shard_policy != TDFS_SHARD_BLOCKED)
    return fail(TDFS_E_INVALID_ARG, "opts.shard_policy");
  if (o->reserved_ != 0) return fail(TDFS_E_INVALID_ARG, "opts.reserved_ must be 0");
  if (o->shared_cursor && (reinterpret_cast<uintptr_t>(o->shared_cursor) & 7u))
    return fail(TDFS_E_INVALID_ARG, "opts.shared_cursor must be 8-byte aligned");
  // leaf stage: a referenced F (lf_byref) is materialised only for a list without a hub bitmap, i.e.
  // of degree <= the smallest hub degree, so it needs no more ids than that; the rest of the shared
  // memory is left to L1 (measured on C2 c4: 845 -> 774 ms with 256 instead of 512 ids per warp)
  L->fcap = kLeafStage;
  if (p->dev.lf_byref && g->n_hubs > 0)
    L->fcap = (int)std::min<int64_t>(kLeafStage, std::max<int64_t>(64, (g->hub_min_deg + 31) / 32 * 32));
  if (o->blocks > 0) {
    L->blocks = o->blocks;
  } else {
    int mn = INT_MAX;
    for (int m = 0; m < 2; m++)
      for (int s = 0; s < 2; s++) {
        int nb = 0;
        int rc = blocks_per_sm(dev, L->wpb, s != 0, m != 0, L->fcap, &nb);
        if (rc) return rc;
        mn = std::min(mn, nb);
      }
    L->blocks = sms * mn;
  }
  const long long n_warps = (long long)L->blocks * L->wpb;
  L->n_levels = std::max(0, p->k - 3);
  const int ints_per_page = o->page_bytes / 4;
  int shift = 0;
  while ((1 << shift) < ints_per_page) shift++;
  L->page_shift = shift;
  // a level holds at most min-operand-length <= d_max candidates
  long long need = std::max<long long>(1, (g->dmax + ints_per_page - 1) / ints_per_page);
  L->E = o->page_table_entries > 0 ? o->page_table_entries : (int)need;
  L->qcap = (uint64_t)(o->queue_ints / 3);
  L->qslots = 1;
  while (L->qslots < L->qcap) L->qslots <<= 1;
  if (o->flags & TDFS_RUN_ARRAY_STACKS) {
    // array-based stacks: every warp-level gets d_max ids (E whole pages) up front (Tables V/VII)
    L->n_pages = (uint64_t)n_warps * L->n_levels * L->E;
  } else if (o->pool_bytes > 0) {
    L->n_pages = (uint64_t)(o->pool_bytes / o->page_bytes);
  } else {
    // every warp-level able to reach d_max, capped at max(4 pages per warp-level, 2 GiB):
    // pages are a per-warp high-water mark, so typical use is ~1 page each
    uint64_t full = (uint64_t)n_warps * L->n_levels * L->E;
    uint64_t floor_pages = std::max<uint64_t>((uint64_t)n_warps * L->n_levels * 4,
                                              (2ull << 30) / (uint64_t)o->page_bytes);
    L->n_pages = std::min(full, floor_pages);
  }
  if (L->n_levels == 0) L->n_pages = 0;
  if (L->n_pages > 0xfffffff0ull) return fail(TDFS_E_INVALID_ARG, "pool too large for 32-bit page ids");
  size_t off = 0;
  L->ctr = off;
  off += align_up(sizeof(unsigned long long) * C_NUM * kCounterStride, 256);
  L->stats = off;
  off += align_up(sizeof(unsigned long long) * S_NUM, 256);
  L->fill = off;
  off += align_up(sizeof(unsigned long long) * kRingChunks, 256);
  L->slots = off;
  off += align_up(sizeof(QSlot) * L->qslots, 256);
  L->tables = off;
  off += align_up(sizeof(uint32_t) * (size_t)n_warps * std::max(L->n_levels, 1) * L->E, 256);
  L->pool = off;
  off += align_up((size_t)L->n_pages * o->page_bytes, 256);
  L->total = off;
  return TDFS_OK;
}

int launch_job(const Graph* g, const Plan* p, const tdfs_run_opts* o, void* ws, size_t ws_bytes, void* stream,
               int mode, int32_t* d_out, uint64_t cap, uint64_t* d_count, bool sync, uint64_t* h_count,
               tdfs_stats* stats, int32_t* h_trace, int64_t trace_cap, int64_t* n_trace, bool ring) {
  WsLayout L;
  int rc = resolve_layout(g, p, o, &L);
  if (rc) return rc;
  if (!ws || ((uintptr_t)ws & 255u)) return fail(TDFS_E_WORKSPACE, "workspace NULL or not 256-byte aligned");
  if (ws_bytes < L.total) return fail(TDFS_E_WORKSPACE, "workspace smaller than tdfs_workspace_bytes()");
  cudaError_t e = cudaSetDevice(g->device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
  cudaStream_t st = (cudaStream_t)stream;
  char* base = (char*)ws;
  const bool want_stats = stats != nullptr;

  KParams P;
  std::memset(&P, 0, sizeof(P));
  P.offs = g->d_offs;
  P.adj = g->d_adj;
  P.src = g->d_src;
  P.label = g->d_label;
  P.n = g->n;
  P.plan = p->dev;
  if (o->flags & TDFS_RUN_NO_REUSE) {
    for (int i = 0; i <= kVF; i++) { P.plan.reuse[i] = -1; P.plan.shortcut[i] &= 2; }
    P.plan.reuse_enabled = 0;
  }
  if (o->flags & TDFS_RUN_NO_SHORTCUT)
    for (int i = 0; i < kMaxK; i++) P.plan.shortcut[i] = 0;
  // lists reused by a later position or the leaf set: a range task over them builds them whole
  P.reused_mask = 0;
  for (int i = 3; i <= kVF; i++)
    if ((i < P.plan.k || i == kVF) && P.plan.reuse[i] >= 2) P.reused_mask |= 1u << P.plan.reuse[i];
  // timeout splits (R30/R33): range tasks at levels 2 .. min(kMaxRangeLevel, k-2); the paper's
  // per-sibling 3-prefix tasks at level 2 only with TDFS_RUN_NO_RANGE_TASKS.  A leaf-level list
  // whose leaves start from its own C(d) (k4: reuse + lf_var) keeps per-sibling tasks at level 2:
  // rebuilding it per range task costs more (measured 86 vs 100 ms).
  P.split_mask = 1u << 2;  // level 2 always (its per-sibling split is the paper's)
  P.range_mask = 0;
  if (!(o->flags & TDFS_RUN_NO_RANGE_TASKS)) {
    for (int d = 2; d <= std::min(kMaxRangeLevel, P.plan.k - 2); d++) {
      const bool leaf_level_reused = d == P.plan.k - 2 && ((P.reused_mask >> d) & 1u) && P.plan.lf_var;
#ifdef TDFS_RANGE_LEAF_REUSED  // build-time experiment: range tasks also for a reused leaf-parent level
      if (true) P.range_mask |= 1u << d;
      (void)leaf_level_reused;
#else
      if (!leaf_level_reused) P.range_mask |= 1u << d;
#endif
    }
    P.split_mask |= P.range_mask;  // deeper levels split only into range tasks
  }
  P.shard_rank = o->shard_rank;
  P.shard_world = o->shard_world;
  P.n_tasks = g->nnz > o->shard_rank ? (g->nnz - o->shard_rank + o->shard_world - 1) / o->shard_world : 0;
  P.gcursor = (unsigned long long*)(base + L.ctr) + C_CURSOR * kCounterStride;
  if (o->shared_cursor) {
    // cross-rank dynamic balancing (NEXT-3): every directed edge, chunks from the shared cursor
    P.shard_rank = 0;
    P.shard_world = 1;
    P.n_tasks = g->nnz;
    P.gcursor = reinterpret_cast<unsigned long long*>(o->shared_cursor);
    P.gshared = 1;
  } else if (o->shard_world > 1 && o->shard_policy == TDFS_SHARD_BLOCKED) {
    // blocks b = rank, rank + W, ... of B edges; the last block of the graph may be partial
    const long long B = TDFS_SHARD_BLOCK_EDGES, nb = (g->nnz + B - 1) / B, W = o->shard_world, r = o->shard_rank;
    const long long mine = nb > r ? (nb - r + W - 1) / W : 0;
    long long nt = mine * B;
    if (mine > 0 && (r + (mine - 1) * W) == nb - 1) nt -= nb * B - g->nnz;  // this rank owns the partial block
    P.n_tasks = nt;
    P.shard_block = (int32_t)B;
  } else if (o->shard_world > 1 && o->shard_policy == TDFS_SHARD_DEGREE_BALANCED) {
    int64_t nt = 0;
    if ((rc = shard_task_list(g, o->shard_rank, o->shard_world, o->shard_policy, &P.task_edges, &nt)) != TDFS_OK)
      return rc;
    P.n_tasks = nt;
  }
  P.chunk = o->chunk;
  P.n_levels = L.n_levels;
  P.slots = (QSlot*)(base + L.slots);
  P.qcap = L.qcap;
  P.qslots = L.qslots;
  P.ctr = (unsigned long long*)(base + L.ctr);
  P.stats = want_stats ? (unsigned long long*)(base + L.stats) : nullptr;
  P.page_tables = (uint32_t*)(base + L.tables);
  P.pool = (int32_t*)(base + L.pool);
  P.n_pages = (uint32_t)L.n_pages;
  P.page_shift = L.page_shift;
  P.E = L.E;
  P.array_stacks = (o->flags & TDFS_RUN_ARRAY_STACKS) ? 1 : 0;
  P.tau_ns = o->tau_ns;
  P.fcap = (o->flags & TDFS_RUN_NO_LEAF_STAGE) ? 0 : L.fcap;
  P.meta_off = (int)smem_meta_offset(L.wpb, L.fcap);
  if (g->d_hub_bits && !(o->flags & TDFS_RUN_NO_HUB_BITMAP)) {
    P.hub_id = g->d_hub_id;
    P.hub_bits = g->d_hub_bits;
    P.hub_words = g->hub_words;
  }
  P.orig = g->d_orig;
  P.out = d_out;
  P.cap = cap;
  if (ring) {
    P.ring_nchunks = kRingChunks;
    P.ring_chunk = cap / kRingChunks;
    P.ring_fill = (unsigned long long*)(base + L.fill);
  }
  int32_t* d_trace = nullptr;
  if (h_trace && trace_cap > 0) {
    if ((e = cudaMalloc(&d_trace, sizeof(int32_t) * 3 * (size_t)trace_cap)) != cudaSuccess)
      return fail(TDFS_E_OOM, "trace buffer");
    P.trace = d_trace;
    P.trace_cap = trace_cap;
  }

  const unsigned long long ticket_base = 0;
  init_counters_kernel<<<1, C_NUM * kCounterStride, 0, st>>>(P.ctr, P.qcap, ticket_base);
  if (want_stats) {
    cudaMemsetAsync(P.stats, 0, sizeof(unsigned long long) * S_NUM, st);
    cudaMemsetAsync(P.stats + S_T_START, 0xff, sizeof(unsigned long long), st);   // min accumulators
    cudaMemsetAsync(P.stats + S_T_EXIT_MIN, 0xff, sizeof(unsigned long long), st);
  }
  if (ring) cudaMemsetAsync(P.ring_fill, 0, sizeof(unsigned long long) * kRingChunks, st);
  {
    int nb = (int)std::min<uint64_t>((L.qslots + 255) / 256, 4096);
    init_queue_kernel<<<std::max(nb, 1), 256, 0, st>>>(P.slots, P.qslots, ticket_base);
  }
  size_t tbytes = sizeof(uint32_t) * (size_t)L.blocks * L.wpb * std::max(L.n_levels, 1) * L.E;
  if (L.n_levels > 0 && !P.array_stacks) cudaMemsetAsync(P.page_tables, 0xff, tbytes, st);
  if (L.n_levels > 0 && P.array_stacks) {
    // array layout: warp-level t owns pages [t*E, (t+1)*E) up front (identity page tables), so no page is
    // ever allocated or found missing during the job; the pool cursor starts exhausted
    const uint64_t nt = (uint64_t)L.blocks * L.wpb * L.n_levels * L.E;
    iota_u32_kernel<<<(int)std::min<uint64_t>((nt + 255) / 256, 65535), 256, 0, st>>>(P.page_tables, nt);
    const unsigned long long np = L.n_pages;
    cudaMemcpyAsync(P.ctr + C_POOL * kCounterStride, &np, sizeof(np), cudaMemcpyHostToDevice, st);
  }

  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  if (want_stats) {
    cudaEventCreate(&ev0);
    cudaEventCreate(&ev1);
    cudaEventRecord(ev0, st);
  }
  KernelFn fn = pick_kernel(mode, want_stats);
  {
    // L1/shared split: ask for just the shared memory this launch's resident blocks need, so the rest of
    // the 256 KB stays L1 (the hub-bitmap and adjacency probes are L1/L2 gathers).  The carveout is a
    // sticky per-function hint: without it a launch inherits the split of an earlier, larger launch.
    int dev = g->device, smem_sm = 0, reserved = 0;
    cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
    cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev);
    int sms = 1;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const long long per_sm_blocks = (L.blocks + sms - 1) / sms;
    const long long need = per_sm_blocks * ((long long)smem_bytes(L.wpb, L.fcap) + reserved);
    if (smem_sm > 0) {
      const int pct = (int)std::min<long long>(100, (need * 100 + smem_sm - 1) / smem_sm);
      cudaFuncSetAttribute(reinterpret_cast<const void*>(fn), cudaFuncAttributePreferredSharedMemoryCarveout, pct);
    }
  }
  fn<<<L.blocks, L.wpb * 32, smem_bytes(L.wpb, L.fcap), st>>>(P);
  if ((e = cudaGetLastError()) != cudaSuccess) {
    cudaFree(d_trace);
    return cuda_fail(e, "kernel launch");
  }
  if (want_stats) cudaEventRecord(ev1, st);
  if (d_count) finalize_kernel<<<1, 32, 0, st>>>(P.ctr, (unsigned long long*)d_count);

  if (!(sync || h_count || want_stats || h_trace)) return TDFS_OK;
  unsigned long long hc[C_NUM * kCounterStride];
  e = cudaMemcpyAsync(hc, P.ctr, sizeof(hc), cudaMemcpyDeviceToHost, st);
  unsigned long long hs[S_NUM];
  if (e == cudaSuccess && want_stats) e = cudaMemcpyAsync(hs, P.stats, sizeof(hs), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) {
    cudaFree(d_trace);
    return cuda_fail(e, "kernel execution");
  }
  if (h_trace && d_trace) {
    long long nt = (long long)hc[C_TRACE * kCounterStride];
    if (n_trace) *n_trace = nt;
    long long ncp = std::min<long long>(nt, trace_cap);
    if (ncp > 0) cudaMemcpy(h_trace, d_trace, sizeof(int32_t) * 3 * (size_t)ncp, cudaMemcpyDeviceToHost);
    cudaFree(d_trace);
  }
  if (want_stats) {
    std::memset(stats, 0, sizeof(*stats));
    for (int i = 0; i < kMaxK + 1; i++) stats->nodes_per_level[i] = hs[S_NODES + i];
    stats->adj_bytes = hs[S_ADJ_BYTES];
    stats->tasks_enqueued = hs[S_ENQ];
    stats->tasks_dequeued = hs[S_DEQ];
    stats->timeouts = hs[S_TIMEOUTS];
    stats->queue_full = hs[S_QFULL];
    stats->edges_scanned = hs[S_EDGES_SCANNED];
    stats->edges_filtered_in = hs[S_EDGES_IN];
    stats->chunks_fetched = hs[S_CHUNKS];
    stats->pages_used = std::min<unsigned long long>(hc[C_POOL * kCounterStride], L.n_pages);
    stats->pool_pages = L.n_pages;
    stats->stream_bytes = hs[S_STREAM];
    if (hs[S_WARPS]) {
      const unsigned long long t0 = hs[S_T_START];
      stats->warp_exit_first_ns = hs[S_T_EXIT_MIN] - t0;
      stats->warp_exit_last_ns = hs[S_T_EXIT_MAX] - t0;
      stats->warp_exit_mean_ns = hs[S_T_EXIT_SUM] / hs[S_WARPS];  // each warp from its own start (~t0)
    }
    stats->grid_blocks = L.blocks;
    stats->warps_per_block = L.wpb;
    stats->page_table_entries = L.E;
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ev0, ev1);
    stats->kernel_ms = ms;
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
  }
  if (hc[C_ERROR * kCounterStride]) return fail(TDFS_E_STACK_EXHAUSTED, "stack page pool or page table exhausted "
                                                "(raise pool_bytes / page_table_entries); no count produced");
  if (h_count) *h_count = hc[C_COUNT * kCounterStride];
  if (mode == 1 && cap < hc[C_COUNT * kCounterStride]) return TDFS_E_OUTPUT_OVERFLOW;
  return TDFS_OK;
}


// Streaming enumerate ("output S"): the kernel writes
// tuples into a device ring of ring_cap tuples (kRingChunks chunks) and waits for free space;
// this host loop copies every full chunk out on a side stream (the DMA engine, concurrent with
// the persistent kernel), hands it to `sink`, zeroes the chunk's fill word and advances the
// consumed counter the kernel waits on; after the kernel ends it drains the last partial chunks.
int stream_job(const Graph* g, const Plan* p, const tdfs_run_opts* o, void* ws, size_t ws_bytes, void* stream,
               int32_t* d_ring, uint64_t ring_cap, SinkFn sink, void* user, uint64_t* n_total) {
  if (!sink || !d_ring || !n_total) return fail(TDFS_E_INVALID_ARG, "enumerate_stream: NULL ring, sink or n_total");
  if (ring_cap < (uint64_t)kRingChunks || ring_cap % kRingChunks)
    return fail(TDFS_E_INVALID_ARG, "enumerate_stream: ring_cap must be a positive multiple of 8");
  const int k = p->k;
  const uint64_t chunk = ring_cap / kRingChunks;
  WsLayout L;
  int rc = resolve_layout(g, p, o, &L);
  if (rc) return rc;
  cudaStream_t st = (cudaStream_t)stream, side = nullptr;
  cudaEvent_t done = nullptr;
  int32_t* host = nullptr;
  unsigned long long* words = nullptr;  // pinned: [0] fill probe, [1] zero, [2] consumed
  cudaError_t e = cudaSetDevice(g->device);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&side, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&done, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaHostAlloc(&host, sizeof(int32_t) * (size_t)(chunk * k), cudaHostAllocDefault);
  if (e == cudaSuccess) e = cudaHostAlloc(&words, 4 * sizeof(unsigned long long), cudaHostAllocDefault);
  auto cleanup = [&]() {
    if (side) cudaStreamDestroy(side);
    if (done) cudaEventDestroy(done);
    if (host) cudaFreeHost(host);
    if (words) cudaFreeHost(words);
  };
  if (e != cudaSuccess) {
    cleanup();
    return cuda_fail(e, "enumerate_stream: setup");
  }
  rc = launch_job(g, p, o, ws, ws_bytes, stream, 1, d_ring, ring_cap, nullptr, false, nullptr, nullptr, nullptr, 0,
                  nullptr, true);
  if (rc) {
    cleanup();
    return rc;
  }
  cudaEventRecord(done, st);
  char* base = (char*)ws;
  unsigned long long* d_fill = (unsigned long long*)(base + L.fill);
  unsigned long long* d_ctr = (unsigned long long*)(base + L.ctr);
  unsigned long long* d_consumed = d_ctr + C_CONSUMED * kCounterStride;
  uint64_t consumed = 0;
  bool aborted = false;
  words[1] = 0;
  auto deliver = [&](uint64_t n) -> cudaError_t {  // copy n tuples at `consumed` out, hand them to sink
    const uint64_t slot = consumed % ring_cap;
    cudaError_t x = cudaMemcpyAsync(host, d_ring + slot * k, sizeof(int32_t) * (size_t)(n * k), cudaMemcpyDeviceToHost, side);
    if (x == cudaSuccess) x = cudaStreamSynchronize(side);
    if (x == cudaSuccess && !aborted && sink(host, n, k, user) != 0) aborted = true;
    return x;
  };
  for (;;) {
    const int c = (int)((consumed / chunk) % kRingChunks);
    e = cudaMemcpyAsync(words, d_fill + c, sizeof(unsigned long long), cudaMemcpyDeviceToHost, side);
    if (e == cudaSuccess) e = cudaStreamSynchronize(side);
    if (e != cudaSuccess) break;
    if (words[0] >= chunk) {  // chunk full: out, then free it for the kernel
      if ((e = deliver(chunk)) != cudaSuccess) break;
      consumed += chunk;
      words[2] = aborted ? (1ull << 62) : consumed;  // abort: nobody waits any more (tuples dropped)
      e = cudaMemcpyAsync(d_fill + c, words + 1, sizeof(unsigned long long), cudaMemcpyHostToDevice, side);
      if (e == cudaSuccess) e = cudaMemcpyAsync(d_consumed, words + 2, sizeof(unsigned long long), cudaMemcpyHostToDevice, side);
      if (e == cudaSuccess) e = cudaStreamSynchronize(side);
      if (e != cudaSuccess) break;
      continue;
    }
    const cudaError_t q = cudaEventQuery(done);
    if (q == cudaSuccess) break;
    if (q != cudaErrorNotReady) { e = q; break; }
    std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
  if (e == cudaSuccess) e = cudaEventSynchronize(done);
  unsigned long long hc[C_NUM * kCounterStride];
  if (e == cudaSuccess) e = cudaMemcpy(hc, d_ctr, sizeof(hc), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) {
    cleanup();
    return cuda_fail(e, "enumerate_stream: kernel execution");
  }
  if (hc[C_ERROR * kCounterStride]) {
    cleanup();
    return fail(TDFS_E_STACK_EXHAUSTED, "stack page pool or page table exhausted; no output");
  }
  const uint64_t total = hc[C_OUTCUR * kCounterStride];
  while (!aborted && consumed < total) {  // the job is over: every reserved slot is written
    const uint64_t n = std::min<uint64_t>(chunk - consumed % chunk, total - consumed);
    if ((e = deliver(n)) != cudaSuccess) break;
    consumed += n;
  }
  cleanup();
  if (e != cudaSuccess) return cuda_fail(e, "enumerate_stream: drain");
  *n_total = total;
  if (aborted) return fail(TDFS_E_INVALID_ARG, "enumerate_stream: the sink aborted (total still exact)");
  return TDFS_OK;
}

}  // namespace tdfs
