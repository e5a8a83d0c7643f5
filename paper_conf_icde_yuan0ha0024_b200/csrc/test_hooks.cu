// Test-only entry points (tdfs_test.h): drive the queue and the paged writer of
// prims.cuh -- the exact device code the matching kernel runs -- in isolation.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstring>
#include <vector>

#include "internal.h"
#include "tdfs_test.h"

namespace tdfs {
namespace {

#include "prims.cuh"

__device__ __forceinline__ Task mk_task(const int32_t* t3) {
  Task k;
  k.hdr = TASK_PREFIX;
  k.v[0] = t3[0];
  k.v[1] = t3[1];
  k.v[2] = t3[2];
  k.v[3] = k.v[4] = k.v[5] = -1;
  return k;
}

// mode 0: one warp fills then drains; mode 1: n warps interleave push/pop then drain.
__global__ void queue_test_kernel(KParams P, int mode, const int32_t* in, long long n_in, int32_t* out,
                                  unsigned long long* n_out, unsigned long long* n_enq) {
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  const Queue q = make_queue(P);
  auto pop_one = [&]() -> bool {
    int got = 0;
    Task k;
    if (lane == 0) got = q_pop(q, k);
    got = __shfl_sync(FULL, got, 0);
    if (got && lane == 0) {
      unsigned long long i = atomicAdd(n_out, 1ull);
      out[3 * i] = k.v[0];
      out[3 * i + 1] = k.v[1];
      out[3 * i + 2] = k.v[2];
    }
    return got != 0;
  };
  if (mode == 0) {
    if (warp != 0) return;
    long long pushed = 0;
    for (long long i = 0; i < n_in; i++) {
      bool ok = q_push_warp(P, q, 1u, mk_task(in + 3 * i), lane);
      if (!ok) break;
      pushed++;
    }
    if (lane == 0) *n_enq = pushed;
    while (pop_one()) {
    }
    return;
  }
  // mode 1
  long long pushed = 0;
  for (long long i = warp; i < n_in; i += nw) {
    // push a batch of up to 32 consecutive tasks of this warp's stride when possible
    bool ok = false;
    while (!ok) {
      ok = q_push_warp(P, q, 1u, mk_task(in + 3 * i), lane);
      if (!ok) pop_one();
    }
    pushed++;
    if ((i / nw) % 2 == 1) pop_one();
  }
  if (lane == 0) atomicAdd(n_enq, (unsigned long long)pushed);
  // drain until all pushes are accounted for
  __syncwarp();
  for (;;) {
    if (pop_one()) continue;
    int done = 0;
    if (lane == 0) {
      __threadfence();
      done = (long long)ld_relaxed_s64(n_out) >= n_in;
    }
    if (__shfl_sync(FULL, done, 0)) break;
    __nanosleep(100);
  }
}

__global__ void paged_test_kernel(KParams P, long long start_pos, unsigned valid_mask, int32_t* page_of_lane,
                                  int32_t* off_of_lane, int32_t* first_new_lane, int32_t* readback_ok) {
  const int lane = threadIdx.x & 31;
  uint32_t* table = P.page_tables;
  // pre-allocate the pages that hold positions < start_pos (a level already filled up to start_pos)
  if (lane == 0) {
    int last = start_pos > 0 ? (int)((start_pos - 1) >> P.page_shift) : -1;
    for (int p = 0; p <= last; p++) ensure_page(P, table, p);
  }
  __syncwarp();
  unsigned long long before = *ctr(P, C_POOL);
  __syncwarp();
  PagedWriter w;
  w.table = table;
  w.cur_p = -1;
  w.cur_pg = NULL_PAGE;
  const bool ok = (valid_mask >> lane) & 1u;
  const int value = 1000000 + lane;
  const unsigned bal = __ballot_sync(FULL, ok);
  bool wr = paged_write(P, w, bal, start_pos, value, lane);
  __syncwarp();
  unsigned long long after = *ctr(P, C_POOL);
  int newpages = (int)(after - before);
  int first_new = -1;
  if (ok && wr) {
    long long pos = start_pos + __popc(bal & lanemask_lt());
    int p = (int)(pos >> P.page_shift);
    page_of_lane[lane] = p;
    off_of_lane[lane] = (int)(pos & ((1ll << P.page_shift) - 1));
    int last_old = start_pos > 0 ? (int)((start_pos - 1) >> P.page_shift) : -1;
    bool on_new = p > last_old;
    unsigned m = __ballot_sync(bal, on_new);
    if (m) first_new = __ffs(m) - 1;
    int rb = paged_read(P, table, pos);
    unsigned good = __ballot_sync(bal, rb == value);
    if (lane == __ffs(bal) - 1) {
      *readback_ok = (good == bal) ? 1 : 0;
      *first_new_lane = first_new;
    }
  } else if (!ok) {
    page_of_lane[lane] = -1;
    off_of_lane[lane] = -1;
  }
  if (lane == 0) {
    if (!wr) *readback_ok = -1;
    if (bal == 0) { *readback_ok = 1; *first_new_lane = -1; }
    page_of_lane[32] = newpages;
  }
}

int cuda_fail(cudaError_t e, const char* what) {
  return fail(TDFS_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

__global__ void init_q(QSlot* slots, unsigned long long cap, unsigned long long nslots, unsigned long long base,
                       unsigned long long* ctrs) {
  for (unsigned long long s = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; s < nslots;
       s += (unsigned long long)gridDim.x * blockDim.x) {
    slots[s].seq = (unsigned)(base + ((s + nslots - (base % nslots)) % nslots));
    slots[s].hdr = -1;
    for (int i = 0; i < 6; i++) slots[s].v[i] = -1;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    ctrs[C_QHEAD * kCounterStride] = base;
    ctrs[C_QTAIL * kCounterStride] = base;
    ctrs[C_QFREE * kCounterStride] = cap;
  }
}

}  // namespace
}  // namespace tdfs

using namespace tdfs;

extern "C" int tdfs_test_queue(int device, int mode, int n_warps, int64_t cap_tasks, uint64_t ticket_base,
                               int64_t n_in, const int32_t* h_in, int32_t* h_out, int64_t* n_out, int64_t* n_enq) {
  if (cap_tasks < 1 || n_in < 0 || (n_in > 0 && (!h_in || !h_out)) || !n_out || !n_enq || n_warps < 1 ||
      (mode != 0 && mode != 1))
    return fail(TDFS_E_INVALID_ARG, "test_queue: bad args");
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) return cuda_fail(e, "test_queue: set device");
  QSlot* slots = nullptr;
  unsigned long long* ctrs = nullptr;
  int32_t *din = nullptr, *dout = nullptr;
  size_t nin = (size_t)std::max<int64_t>(n_in, 1);
  unsigned long long nslots = 1;
  while (nslots < (unsigned long long)cap_tasks) nslots <<= 1;
  e = cudaMalloc(&slots, sizeof(QSlot) * (size_t)nslots);
  if (e == cudaSuccess) e = cudaMalloc(&ctrs, sizeof(unsigned long long) * (C_NUM * kCounterStride + 2));
  if (e == cudaSuccess) e = cudaMalloc(&din, sizeof(int32_t) * 3 * nin);
  if (e == cudaSuccess) e = cudaMalloc(&dout, sizeof(int32_t) * 3 * nin);
  if (e != cudaSuccess) {
    cudaFree(slots); cudaFree(ctrs); cudaFree(din); cudaFree(dout);
    return fail(TDFS_E_OOM, "test_queue: alloc");
  }
  cudaMemset(ctrs, 0, sizeof(unsigned long long) * (C_NUM * kCounterStride + 2));
  if (n_in) cudaMemcpy(din, h_in, sizeof(int32_t) * 3 * n_in, cudaMemcpyHostToDevice);
  init_q<<<64, 256>>>(slots, (unsigned long long)cap_tasks, nslots, ticket_base, ctrs);
  KParams P;
  std::memset(&P, 0, sizeof(P));
  P.slots = slots;
  P.qcap = (uint64_t)cap_tasks;
  P.qslots = nslots;
  P.ctr = ctrs;
  unsigned long long* d_nout = ctrs + C_NUM * kCounterStride;
  unsigned long long* d_nenq = d_nout + 1;
  int threads = 32 * std::min(n_warps, 4);
  int blocks = (n_warps * 32 + threads - 1) / threads;
  queue_test_kernel<<<blocks, threads>>>(P, mode, din, n_in, dout, d_nout, d_nenq);
  e = cudaDeviceSynchronize();
  unsigned long long h2[2] = {0, 0};
  if (e == cudaSuccess) e = cudaMemcpy(h2, d_nout, sizeof(h2), cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && h2[0] > 0)
    e = cudaMemcpy(h_out, dout, sizeof(int32_t) * 3 * std::min<unsigned long long>(h2[0], nin), cudaMemcpyDeviceToHost);
  cudaFree(slots); cudaFree(ctrs); cudaFree(din); cudaFree(dout);
  if (e != cudaSuccess) return cuda_fail(e, "test_queue: run");
  *n_out = (int64_t)h2[0];
  *n_enq = (int64_t)h2[1];
  return TDFS_OK;
}

extern "C" int tdfs_test_paged_write(int device, int page_bytes, int64_t start_pos, uint32_t valid_mask,
                                     int32_t* h_page_of_lane, int32_t* h_offset_of_lane, int32_t* n_new_pages,
                                     int32_t* first_lane_on_new_page, int32_t* readback_ok) {
  if (page_bytes < 128 || (page_bytes & (page_bytes - 1)) || start_pos < 0 || !h_page_of_lane || !h_offset_of_lane ||
      !n_new_pages || !first_lane_on_new_page || !readback_ok)
    return fail(TDFS_E_INVALID_ARG, "test_paged_write: bad args");
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) return cuda_fail(e, "test_paged_write: set device");
  int ints = page_bytes / 4, shift = 0;
  while ((1 << shift) < ints) shift++;
  int E = (int)((start_pos + 32) / ints) + 2;
  uint32_t* table = nullptr;
  int32_t* pool = nullptr;
  unsigned long long* ctrs = nullptr;
  int32_t* dres = nullptr;
  e = cudaMalloc(&table, sizeof(uint32_t) * E);
  if (e == cudaSuccess) e = cudaMalloc(&pool, (size_t)page_bytes * E);
  if (e == cudaSuccess) e = cudaMalloc(&ctrs, sizeof(unsigned long long) * C_NUM * kCounterStride);
  if (e == cudaSuccess) e = cudaMalloc(&dres, sizeof(int32_t) * 70);
  if (e != cudaSuccess) {
    cudaFree(table); cudaFree(pool); cudaFree(ctrs); cudaFree(dres);
    return fail(TDFS_E_OOM, "test_paged_write: alloc");
  }
  cudaMemset(table, 0xff, sizeof(uint32_t) * E);
  cudaMemset(ctrs, 0, sizeof(unsigned long long) * C_NUM * kCounterStride);
  cudaMemset(dres, 0xff, sizeof(int32_t) * 70);
  KParams P;
  std::memset(&P, 0, sizeof(P));
  P.ctr = ctrs;
  P.page_tables = table;
  P.pool = pool;
  P.n_pages = (uint32_t)E;
  P.page_shift = shift;
  P.E = E;
  paged_test_kernel<<<1, 32>>>(P, start_pos, valid_mask, dres, dres + 33, dres + 66, dres + 67);
  int32_t h[70];
  e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(h, dres, sizeof(h), cudaMemcpyDeviceToHost);
  cudaFree(table); cudaFree(pool); cudaFree(ctrs); cudaFree(dres);
  if (e != cudaSuccess) return cuda_fail(e, "test_paged_write: run");
  for (int i = 0; i < 32; i++) {
    h_page_of_lane[i] = h[i];
    h_offset_of_lane[i] = h[33 + i];
  }
  *n_new_pages = h[32];
  *first_lane_on_new_page = h[66];
  *readback_ok = h[67];
  return TDFS_OK;
}
