// l2peak.cu -- measured L2 read bandwidth of this B200 (the secondary roofline of DESIGN.md §5.4):
// every block reads a buffer that fits in L2 (after a warm-up pass) with 16-byte loads, many times.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o l2peak scripts/l2peak.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_read(const uint4* __restrict__ p, size_t n, int reps, unsigned long long* sink) {
  unsigned acc = 0;
  for (int r = 0; r < reps; r++)
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
      const uint4 v = __ldcg(p + i);  // L2 (bypass L1)
      acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
  if (acc == 0x12345678u) atomicAdd(sink, 1ull);
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (size_t mb : {16, 32, 64}) {
    const size_t bytes = mb << 20, n = bytes / 16;
    uint4* p;
    unsigned long long* sink;
    cudaMalloc(&p, bytes);
    cudaMalloc(&sink, 8);
    cudaMemset(p, 1, bytes);
    const int reps = 20;
    k_read<<<sms * 8, 512>>>(p, n, 1, sink);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int t = 0; t < 5; t++) {
      cudaEventRecord(a);
      k_read<<<sms * 8, 512>>>(p, n, reps, sink);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (ms < best) best = ms;
    }
    printf("{\"buffer_mb\": %zu, \"l2_read_gbs\": %.1f}\n", mb, (double)bytes * reps / (best * 1e-3) / 1e9);
    cudaFree(p);
    cudaFree(sink);
  }
  return 0;
}
