// L2 read-bandwidth microbenchmark (measurement tooling, not the product): every SM streams a
// 48 MB buffer (L2-resident after the first pass, B200 L2 = 126 MB) with 128-bit loads, many
// passes; bytes read / CUDA-event time = the L2 peak the roofline's "l2" object divides by.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o l2_peak scripts/l2_peak.cu && ./l2_peak
#include <cstdio>
#include <cuda_runtime.h>

__global__ void l2_read(const int4* __restrict__ a, long long n4, int passes, int* out) {
  int acc = 0;
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (int p = 0; p < passes; p++)
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) {
      const int4 v = __ldcg(a + ((i + (long long)p * 4099) % n4));  // .cg: L2, not L1
      acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
  if (acc == 0x7fffffff) out[0] = acc;
}

int main() {
  const long long bytes = 48ll << 20, n4 = bytes / 16;
  int4* a;
  int* o;
  cudaMalloc(&a, bytes);
  cudaMalloc(&o, 4);
  cudaMemset(a, 1, bytes);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int passes = 40;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  double best = 0;
  for (int rep = 0; rep < 6; rep++) {
    l2_read<<<sms * 4, 512>>>(a, n4, 1, o);  // warm L2
    cudaEventRecord(e0);
    l2_read<<<sms * 4, 512>>>(a, n4, passes, o);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    const double gbs = (double)bytes * passes / (ms / 1e3) / 1e9;
    if (gbs > best) best = gbs;
  }
  printf("{\"l2_read_peak_gbs\": %.1f, \"buffer_mb\": 48, \"passes\": %d, \"sms\": %d}\n", best, passes, sms);
  return 0;
}
