// Microbenchmark: event span of an empty 148 x 320 grid with 217 KB of dynamic shared
// memory (the snapshot kernels' launch shape) when the kernel before it on the stream
// (a) has the same shape, (b) uses no shared memory (a plain elementwise kernel, like
// the L2 flush or an application kernel), (c) as (b) with both kernels preferring the
// maximum shared-memory carveout. Tells whether the L1/shared reconfiguration between
// kernels is part of the per-launch fixed cost. Not part of the library.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__global__ void big(int* sink) {
  extern __shared__ __align__(128) uint8_t sm[];
  sm[threadIdx.x] = (uint8_t)threadIdx.x;
  __syncthreads();
  if (sm[(threadIdx.x * 7) & 255] == 255 && sink) *sink = 1;
}
__global__ void small(float* p, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) p[i] = p[i] * 0.5f + 1.f;
}

int main() {
  const size_t smem = 217 * 1024;
  cudaFuncSetAttribute(big, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  float* buf;
  cudaMalloc(&buf, 64 << 20);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaStream_t s;
  cudaStreamCreate(&s);
  for (int mode = 0; mode < 3; ++mode) {
    if (mode == 2) {
      cudaFuncSetAttribute(big, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
      cudaFuncSetAttribute(small, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    }
    float tot = 0, mn = 1e9;
    const int reps = 50;
    for (int r = 0; r < reps + 5; ++r) {
      if (mode == 0)
        big<<<148, 320, smem, s>>>(nullptr);
      else
        small<<<1184, 256, 0, s>>>(buf, 16 << 20);
      cudaEventRecord(a, s);
      big<<<148, 320, smem, s>>>(nullptr);
      cudaEventRecord(b, s);
      cudaStreamSynchronize(s);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (r >= 5) {
        tot += ms;
        mn = ms < mn ? ms : mn;
      }
    }
    printf("mode %d (%s): mean %.2f us min %.2f us\n", mode,
           mode == 0 ? "after the same shape" : mode == 1 ? "after a no-smem kernel" : "after it, max carveout both",
           tot / reps * 1e3, mn * 1e3);
  }
  return 0;
}
