// Microbenchmark: copy throughput with cp.async.bulk (TMA 1D) per warp: each warp
// streams a contiguous stretch in tiles of T bytes, NT tiles in flight, one elected
// lane issuing bulk load (mbarrier) and bulk store per tile. Prints GB/s (2S).
// usage: tma_copy  (sweeps W warps/CTA, T tile bytes, NT tiles)
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int NT>
__global__ void k(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst, size_t n, int T) {
  extern __shared__ __align__(128) uint8_t sm[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  uint8_t* tiles = sm + (size_t)warp * NT * T;
  uint64_t* mb = reinterpret_cast<uint64_t*>(sm + (size_t)nw * NT * T) + warp * NT;
  if (lane == 0) {
    for (int t = 0; t < NT; ++t) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(mb + t)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncwarp();
  const size_t gw = (size_t)blockIdx.x * nw + warp, tw = (size_t)gridDim.x * nw;
  const size_t ntiles = n / T, per = (ntiles + tw - 1) / tw;
  const size_t t0 = gw * per, t1 = t0 + per < ntiles ? t0 + per : ntiles;
  if (lane != 0 || t0 >= t1) return;
  uint32_t phase = 0;
  auto issue = [&](size_t i) {
    const int t = (int)(i % NT);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(mb + t)), "r"(T));
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     sa(tiles + t * T)),
                 "l"(src + i * T), "r"(T), "r"(sa(mb + t))
                 : "memory");
  };
  for (size_t i = t0; i < t1 && i < t0 + NT; ++i) issue(i);
  for (size_t i = t0; i < t1; ++i) {
    const int t = (int)(i % NT);
    asm volatile(
        "{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}" ::"r"(
            sa(mb + t)),
        "r"((phase >> t) & 1u)
        : "memory");
    phase ^= 1u << t;
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + i * T), "r"(sa(tiles + t * T)),
                 "r"(T)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;");
    if (i + NT < t1) {
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      issue(i + NT);
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

template <int NT>
void run(const uint8_t* s, uint8_t* d, size_t n, int W, int T, int sms) {
  const size_t smem = (size_t)W * NT * T + W * NT * 8 + 16;
  if (smem > 227 * 1024) return;
  cudaFuncSetAttribute(k<NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  k<NT><<<sms, W * 32, smem>>>(s, d, n, T);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e9;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(a);
    k<NT><<<sms, W * 32, smem>>>(s, d, n, T);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    best = ms < best ? ms : best;
  }
  printf("W=%2d T=%5d NT=%d: %7.1f GB/s (2S)  err=%s\n", W, T, NT, 2.0 * n / (best * 1e-3) / 1e9,
         cudaGetErrorString(cudaGetLastError()));
}

int main(int argc, char** argv) {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t n = argc > 1 ? (size_t)atoll(argv[1]) : (1ull << 31);
  uint8_t *s, *d;
  cudaMalloc(&s, n);
  cudaMalloc(&d, n);
  cudaMemset(s, 1, n);
  for (int W : {4, 8, 16})
    for (int T : {4096, 4608, 8192, 16384}) {
      run<2>(s, d, n, W, T, sms);
      run<3>(s, d, n, W, T, sms);
      run<4>(s, d, n, W, T, sms);
    }
  return 0;
}
