// Microbenchmark: copy throughput for work-distribution patterns, 16 warps/SM,
// one CTA per SM. (a) grid-stride blocks of U*512 B; (b) warp-private 64 KiB chunks
// walked sequentially in rounds of U*512 B; (c) like (b) with the next round's
// loads issued before the current round's stores (our kernel's skeleton).
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint4 ldna(const uint4* p) {
  uint4 r;
  asm("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

template <int U, int MODE, int G = 1>
__global__ void k(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n16) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const size_t gw = (size_t)blockIdx.x * nw + warp, tw = (size_t)gridDim.x * nw;
  const size_t blk = (size_t)U * 32;
  if (MODE == 0) {
    for (size_t b = gw; b * blk < n16; b += tw) {
      uint4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = ldna(src + b * blk + u * 32 + lane);
#pragma unroll
      for (int u = 0; u < U; ++u) dst[b * blk + u * 32 + lane] = v[u];
    }
  } else if (MODE == 3) {
    // groups of G warps share a chunk; warp q of a group copies rounds [q*R/G, (q+1)*R/G)
    const size_t chunk16 = 65536 / 16, rounds = chunk16 / blk, per = rounds / G;
    const size_t grp = gw / G, ngrp = tw / G, q = gw % G;
    for (size_t c = grp; c * chunk16 < n16; c += ngrp) {
      const uint4* s = src + c * chunk16 + q * per * blk;
      uint4* d = dst + c * chunk16 + q * per * blk;
      uint4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = ldna(s + u * 32 + lane);
      for (size_t r = 0; r < per; ++r) {
#pragma unroll
        for (int u = 0; u < U; ++u) d[r * blk + u * 32 + lane] = v[u];
        if (r + 1 < per) {
#pragma unroll
          for (int u = 0; u < U; ++u) v[u] = ldna(s + (r + 1) * blk + u * 32 + lane);
        }
      }
    }
  } else {
    const size_t chunk16 = 65536 / 16, rounds = chunk16 / blk;
    for (size_t c = gw; c * chunk16 < n16; c += tw) {
      const uint4* s = src + c * chunk16;
      uint4* d = dst + c * chunk16;
      uint4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = ldna(s + u * 32 + lane);
      for (size_t r = 0; r < rounds; ++r) {
        if (MODE == 1) {
#pragma unroll
          for (int u = 0; u < U; ++u) d[r * blk + u * 32 + lane] = v[u];
          if (r + 1 < rounds) {
#pragma unroll
            for (int u = 0; u < U; ++u) v[u] = ldna(s + (r + 1) * blk + u * 32 + lane);
          }
        } else {
          uint4 w[U];
          if (r + 1 < rounds) {
#pragma unroll
            for (int u = 0; u < U; ++u) w[u] = ldna(s + (r + 1) * blk + u * 32 + lane);
          }
#pragma unroll
          for (int u = 0; u < U; ++u) d[r * blk + u * 32 + lane] = v[u];
#pragma unroll
          for (int u = 0; u < U; ++u) v[u] = w[u];
        }
      }
    }
  }
}

template <int U, int MODE, int G = 1>
void run(int sms, const uint4* a, uint4* b, size_t n16) {
  auto kk = k<U, MODE, G>;
  const int smem = 200 * 1024;
  cudaFuncSetAttribute(kk, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  kk<<<sms, 512, smem>>>(a, b, n16);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) kk<<<sms, 512, smem>>>(a, b, n16);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  printf("mode=%d G=%2d U=%2d  %.0f GB/s (2S)  err=%s\n", MODE, G, U, 2.0 * n16 * 16 * 5 / (ms * 1e-3) / 1e9,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t bytes = 463ull << 20, n16 = bytes / 16;
  uint4 *a, *b;
  cudaMalloc(&a, bytes);
  cudaMalloc(&b, bytes);
  cudaMemset(a, 1, bytes);
  run<4, 0>(sms, a, b, n16);
  run<8, 0>(sms, a, b, n16);
  run<4, 1>(sms, a, b, n16);
  run<8, 1>(sms, a, b, n16);
  run<4, 2>(sms, a, b, n16);
  run<8, 2>(sms, a, b, n16);
  run<8, 3, 2>(sms, a, b, n16);
  run<8, 3, 4>(sms, a, b, n16);
  run<8, 3, 8>(sms, a, b, n16);
  run<8, 3, 16>(sms, a, b, n16);
  run<4, 3, 4>(sms, a, b, n16);
  return 0;
}
