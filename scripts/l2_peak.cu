// L2 microbenchmarks (measurement tooling, not the product) -- the denominators of the "l2" roofline:
//  (1) stream: every SM re-reads an L2-resident buffer with 128-bit .cg loads (8 independent loads per
//      thread in flight), bytes / CUDA-event time;
//  (2) random sectors: every thread reads 4 B from pseudo-random 32-B sectors of an L2-resident buffer
//      (8 independent .cg loads in flight per thread) -- the access pattern of the matching kernel's
//      bitmap and binary-search probes; reported as sectors/ns and as sector bytes/s.
// Buffers of 24 and 48 MB (B200 L2 = 126 MB in two partitions); the best of 6 repetitions each.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o l2_peak scripts/l2_peak.cu && ./l2_peak
#include <cstdio>
#include <cuda_runtime.h>

__global__ void l2_stream(const int4* __restrict__ a, long long n4, int passes, int* out) {
  int acc = 0;
  const long long stride = (long long)gridDim.x * blockDim.x;
  const long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  for (int p = 0; p < passes; p++)
    for (long long i = t; i + 7 * stride < n4; i += 8 * stride) {
      int4 v[8];
#pragma unroll
      for (int u = 0; u < 8; u++) v[u] = __ldcg(a + i + u * stride);
#pragma unroll
      for (int u = 0; u < 8; u++) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
  if (acc == 0x7fffffff) out[0] = acc;
}

__device__ __forceinline__ unsigned hash32(unsigned x) {
  x ^= x >> 16;
  x *= 0x7feb352du;
  x ^= x >> 15;
  x *= 0x846ca68bu;
  x ^= x >> 16;
  return x;
}

// n_sect a power of two; each load touches one 32-B sector (8 ints)
__global__ void l2_random(const int* __restrict__ a, unsigned n_sect, int iters, int* out) {
  int acc = 0;
  const unsigned t = blockIdx.x * blockDim.x + threadIdx.x;
  for (int it = 0; it < iters; it++) {
    int v[8];
#pragma unroll
    for (int u = 0; u < 8; u++) {
      const unsigned s = hash32(t * 0x9e3779b9u + (unsigned)(it * 8 + u)) & (n_sect - 1);
      v[u] = __ldcg(a + (size_t)s * 8 + (t & 7));
    }
#pragma unroll
    for (int u = 0; u < 8; u++) acc ^= v[u];
  }
  if (acc == 0x7fffffff) out[0] = acc;
}

int main() {
  int* o;
  cudaMalloc(&o, 4);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  double best_stream = 0, best_rand = 0;
  int best_stream_mb = 0, best_rand_mb = 0;
  for (int mb : {24, 48}) {
    const long long bytes = (long long)mb << 20, n4 = bytes / 16;
    int4* a;
    cudaMalloc(&a, bytes);
    cudaMemset(a, 1, bytes);
    const int passes = 40;
    for (int rep = 0; rep < 6; rep++) {
      l2_stream<<<sms * 8, 256>>>(a, n4, 1, o);  // warm L2
      cudaEventRecord(e0);
      l2_stream<<<sms * 8, 256>>>(a, n4, passes, o);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      const long long per_pass = (n4 / (8ll * sms * 8 * 256)) * (8ll * sms * 8 * 256) * 16;  // bytes the loop reads
      const double gbs = (double)per_pass * passes / (ms / 1e3) / 1e9;
      if (gbs > best_stream) { best_stream = gbs; best_stream_mb = mb; }
    }
    const unsigned n_sect = (unsigned)(bytes / 32);
    const int iters = 256, blocks = sms * 8, threads = 256;
    for (int rep = 0; rep < 6; rep++) {
      l2_random<<<blocks, threads>>>(reinterpret_cast<int*>(a), n_sect, 16, o);
      cudaEventRecord(e0);
      l2_random<<<blocks, threads>>>(reinterpret_cast<int*>(a), n_sect, iters, o);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      const double sect_per_ns = (double)blocks * threads * iters * 8 / (ms * 1e6);
      if (sect_per_ns > best_rand) { best_rand = sect_per_ns; best_rand_mb = mb; }
    }
    cudaFree(a);
  }
  printf("{\"l2_read_peak_gbs\": %.1f, \"stream_buffer_mb\": %d, \"l2_random_sectors_per_ns\": %.1f, "
         "\"l2_random_sector_gbs\": %.1f, \"random_buffer_mb\": %d, \"sms\": %d}\n",
         best_stream, best_stream_mb, best_rand, best_rand * 32.0, best_rand_mb, sms);
  return 0;
}
