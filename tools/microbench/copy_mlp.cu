// Microbenchmark: copy throughput vs warps per SM and 16-B loads in flight per
// lane, one CTA per SM (large dynamic smem forces it). Not part of the library.
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

template <int U>
__global__ void copyk(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n16, int smem_dummy) {
  extern __shared__ uint4 sm[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const size_t gw = (size_t)blockIdx.x * nw + warp, tw = (size_t)gridDim.x * nw;
  const size_t blk = (size_t)U * 32;  // granules per warp-iteration
  for (size_t b = gw; b * blk < n16; b += tw) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      size_t i = b * blk + u * 32 + lane;
      asm("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(src + i));
    }
#pragma unroll
    for (int u = 0; u < U; ++u) dst[b * blk + u * 32 + lane] = v[u];
  }
  if (smem_dummy < 0) sm[threadIdx.x] = make_uint4(0, 0, 0, 0);
}

template <int U>
void run(int warps, int sms, const uint4* a, uint4* b, size_t n16, size_t smem) {
  auto k = copyk<U>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  k<<<sms, warps * 32, smem>>>(a, b, n16, 0);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) k<<<sms, warps * 32, smem>>>(a, b, n16, 0);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  printf("warps=%2d U=%2d inflight/SM=%4d KiB  %.0f GB/s (2S)\n", warps, U, warps * U * 512 / 1024,
         2.0 * n16 * 16 * 5 / (ms * 1e-3) / 1e9);
}

int main(int argc, char** argv) {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t bytes = argc > 1 ? (size_t)atoll(argv[1]) : (1ull << 30), n16 = bytes / 16;
  uint4 *a, *b;
  cudaMalloc(&a, bytes);
  cudaMalloc(&b, bytes);
  cudaMemset(a, 1, bytes);
  const size_t smem = 200 * 1024;
  for (int w : {8, 16, 24, 32}) {
    run<4>(w, sms, a, b, n16, smem);
    run<8>(w, sms, a, b, n16, smem);
    run<16>(w, sms, a, b, n16, smem);
  }
  run<4>(64, sms, a, b, n16, 16 * 1024);
  run<8>(48, sms, a, b, n16, 16 * 1024);
  return 0;
}
