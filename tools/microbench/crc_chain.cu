// Microbenchmark: throughput of the lane-private slicing-by-4 CRC chain alone
// (data already in shared memory), as a function of warps per CTA and the number
// of independent chains per lane. Prints B/clk/SM. Not part of the library.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int CH>
__global__ void chain(uint32_t* out, int iters) {
  extern __shared__ __align__(16) uint32_t smem[];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 32768; i += blockDim.x) smem[i] = i * 2654435761u;
  __syncthreads();
  const uint8_t* tb = reinterpret_cast<const uint8_t*>(smem);
  const uint32_t l4 = lane * 4;
  uint32_t crc[CH];
  for (int c = 0; c < CH; ++c) crc[c] = threadIdx.x + c;
  uint32_t w = blockIdx.x;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int c = 0; c < CH; ++c) {
      const uint32_t x = crc[c] ^ (w + c);
      crc[c] = *(const uint32_t*)(tb + __byte_perm(x, l4, 0x5504)) ^ *(const uint32_t*)(tb + 128 + __byte_perm(x, l4, 0x5514)) ^
               *(const uint32_t*)(tb + 65536 + __byte_perm(x, l4, 0x5524)) ^ *(const uint32_t*)(tb + 65536 + 128 + __byte_perm(x, l4, 0x5534));
    }
    w += 0x9E3779B9u;
  }
  uint32_t r = 0;
  for (int c = 0; c < CH; ++c) r ^= crc[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = r;
}

template <int CH>
void run(int warps, int sms) {
  const int iters = 4096;
  uint32_t* out;
  cudaMalloc(&out, sms * warps * 32 * 4);
  auto k = chain<CH>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 131072);
  k<<<sms, warps * 32, 131072>>>(out, 16);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  k<<<sms, warps * 32, 131072>>>(out, iters);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double bytes = (double)sms * warps * 32 * iters * 4 * CH;
  double cycles = ms * 1e-3 * clk * 1e3;
  printf("chains=%d warps=%2d  %.2f B/clk/SM  (%.0f GB/s chip)\n", CH, warps, bytes / cycles / sms, bytes / ms / 1e6);
  cudaFree(out);
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int w : {4, 8, 16, 24, 32}) run<1>(w, sms);
  for (int w : {4, 8, 16, 24, 32}) run<2>(w, sms);
  for (int w : {4, 8, 16, 32}) run<4>(w, sms);
  return 0;
}
