// Microbenchmark: event-timed cost of launching an empty persistent grid (148 CTAs x
// 320 threads, 217 KB dynamic smem) from an idle GPU, with and without a 135 KB
// bulk-copied table prologue, to separate the fixed per-launch cost of the
// snapshot kernels from their streaming time. Not part of the library.
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <bool kTables>
__global__ void k(const uint8_t* tab, uint32_t bytes, int* sink) {
  extern __shared__ __align__(128) uint8_t sm[];
  if (kTables) {
    __shared__ uint64_t mb;
    if (threadIdx.x == 0) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&mb)));
      asm volatile("fence.mbarrier_init.release.cluster;");
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&mb)), "r"(bytes));
      for (uint32_t o = 0; o < bytes; o += 32768) {
        const uint32_t n = bytes - o < 32768 ? bytes - o : 32768;
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         sa(sm + o)),
                     "l"(tab + o), "r"(n), "r"(sa(&mb))
                     : "memory");
      }
    }
    __syncthreads();
    asm volatile(
        "{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra W_%=;\n}" ::"r"(
            sa(&mb))
        : "memory");
    if (sm[threadIdx.x * 7] == 123 && sink) *sink = 1;
  }
}

int main() {
  const size_t smem = 217 * 1024;
  uint8_t* tab;
  cudaMalloc(&tab, 256 * 1024);
  cudaMemset(tab, 1, 256 * 1024);
  cudaFuncSetAttribute(k<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int mode = 0; mode < 4; ++mode) {
    float tot = 0, mn = 1e9;
    for (int r = 0; r < 20; ++r) {
      cudaDeviceSynchronize();
      cudaEventRecord(a);
      if (mode == 0) k<false><<<148, 320, smem>>>(tab, 0, nullptr);
      if (mode == 1) k<true><<<148, 320, smem>>>(tab, 135680, nullptr);
      if (mode == 2) k<false><<<148, 320, 0>>>(tab, 0, nullptr);
      if (mode == 3) {  // two back-to-back: the second's cost without host launch latency
        k<true><<<148, 320, smem>>>(tab, 135680, nullptr);
        k<true><<<148, 320, smem>>>(tab, 135680, nullptr);
      }
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (r >= 5) tot += ms, mn = ms < mn ? ms : mn;
    }
    const char* name[] = {"empty 217KB smem", "135KB table prologue", "empty no smem", "2x table prologue"};
    printf("%-22s mean %.2f us  min %.2f us\n", name[mode], tot / 15 * 1e3, mn * 1e3);
  }
  // graph of [event a, kernel, event b]: the GPU receives the three together, so the
  // span no longer contains the host's launch latency. Host cost measured per call:
  // (g) launch only, (u) kernel-node parameter + both event updates, then launch.
  {
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaGraph_t g;
    cudaGraphCreate(&g, 0);
    cudaGraphNode_t na, nk, nb;
    cudaGraphAddEventRecordNode(&na, g, nullptr, 0, a);
    const uint8_t* tp = tab;
    uint32_t by = 135680;
    int* sk = nullptr;
    void* args[] = {&tp, &by, &sk};
    cudaKernelNodeParams kp = {};
    kp.func = (void*)k<true>;
    kp.gridDim = dim3(148);
    kp.blockDim = dim3(320);
    kp.sharedMemBytes = (unsigned)smem;
    kp.kernelParams = args;
    cudaGraphAddKernelNode(&nk, g, &na, 1, &kp);
    cudaGraphAddEventRecordNode(&nb, g, &nk, 1, b);
    cudaGraphExec_t ge;
    cudaGraphInstantiate(&ge, g, 0);
    cudaEvent_t a2, b2;
    cudaEventCreate(&a2);
    cudaEventCreate(&b2);
    for (int mode = 0; mode < 3; ++mode) {
      float tot = 0, mn = 1e9;
      double host = 0;
      for (int r = 0; r < 40; ++r) {
        cudaDeviceSynchronize();
        auto t0 = std::chrono::steady_clock::now();
        cudaEvent_t ea = a, eb = b;
        if (mode == 0) {
          cudaGraphLaunch(ge, s);
        } else if (mode == 1) {
          ea = (r & 1) ? a2 : a, eb = (r & 1) ? b2 : b;
          cudaGraphExecKernelNodeSetParams(ge, nk, &kp);
          cudaGraphExecEventRecordNodeSetEvent(ge, na, ea);
          cudaGraphExecEventRecordNodeSetEvent(ge, nb, eb);
          cudaGraphLaunch(ge, s);
        } else {
          cudaEventRecord(a, s);
          k<true><<<148, 320, smem, s>>>(tab, 135680, nullptr);
          cudaEventRecord(b, s);
        }
        auto t1 = std::chrono::steady_clock::now();
        cudaEventSynchronize(eb);
        float ms;
        cudaEventElapsedTime(&ms, ea, eb);
        if (r >= 10) tot += ms, mn = ms < mn ? ms : mn, host += std::chrono::duration<double, std::micro>(t1 - t0).count();
      }
      // host cost of reading the span back (cudaEventElapsedTime after completion)
      {
        auto q0 = std::chrono::steady_clock::now();
        float x = 0;
        for (int i = 0; i < 100; ++i) cudaEventElapsedTime(&x, mode == 1 ? a2 : a, mode == 1 ? b2 : b);
        auto q1 = std::chrono::steady_clock::now();
        printf("  cudaEventElapsedTime after mode %d: %.2f us/call\n", mode,
               std::chrono::duration<double, std::micro>(q1 - q0).count() / 100);
      }
      const char* name[] = {"graph [ev,k,ev]", "graph + node updates", "stream record/launch/record"};
      printf("%-28s span mean %.2f us  min %.2f us  host %.2f us/call\n", name[mode], tot / 30 * 1e3, mn * 1e3,
             host / 30);
    }
  }
  return 0;
}
