// Microbenchmark: how fast can the host get N bytes of pinned memory?
//  (a) cudaHostAlloc; (b) posix_memalign + touch on T threads + one cudaHostRegister;
//  (c) posix_memalign + touch + cudaHostRegister of T pieces on T threads;
//  (d) like (c) with MADV_HUGEPAGE; (e) like (b) with MADV_HUGEPAGE. Then a D2H copy into each to check it is usable at
//  pinned speed. Not part of the library.
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <sys/mman.h>
#include <thread>
#include <vector>
#include <cuda_runtime.h>

static double now() { return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count(); }

static double d2h_gbs(void* h, void* d, size_t n) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaMemcpy(h, d, n, cudaMemcpyDeviceToHost);
  cudaEventRecord(a);
  cudaMemcpyAsync(h, d, n, cudaMemcpyDeviceToHost);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  return n / (ms * 1e-3) / 1e9;
}

int main(int argc, char** argv) {
  const size_t n = (argc > 1 ? strtoull(argv[1], 0, 10) : 4ull) << 30;
  const int T = argc > 2 ? atoi(argv[2]) : 8;
  void* d;
  cudaMalloc(&d, n);
  cudaFree(0);
  {
    double t0 = now();
    void* h;
    cudaHostAlloc(&h, n, cudaHostAllocDefault);
    double t1 = now();
    printf("(a) cudaHostAlloc %zu MiB: %.3f s (%.2f GB/s)  D2H %.1f GB/s\n", n >> 20, t1 - t0, n / (t1 - t0) / 1e9,
           d2h_gbs(h, d, n));
    cudaFreeHost(h);
  }
  for (int mode = 0; mode < 4; ++mode) {
    double t0 = now();
    void* h = nullptr;
    if (posix_memalign(&h, 2 << 20, n)) return 1;
    if (mode >= 2) madvise(h, n, MADV_HUGEPAGE);
    const size_t piece = (n / T + 4095) & ~(size_t)4095;
    std::vector<std::thread> th;
    for (int t = 0; t < T; ++t)
      th.emplace_back([=] {
        char* p = (char*)h + t * piece;
        size_t m = (size_t)t * piece >= n ? 0 : std::min(piece, n - (size_t)t * piece);
        for (size_t o = 0; o < m; o += 4096) p[o] = 0;
        if ((mode == 1 || mode == 2) && m) cudaHostRegister(p, m, cudaHostRegisterDefault);
      });
    for (auto& x : th) x.join();
    if (mode == 0 || mode == 3) cudaHostRegister(h, n, cudaHostRegisterDefault);
    double t1 = now();
    printf("(%c) memalign + touch x%d + %s%s: %.3f s (%.2f GB/s)  D2H %.1f GB/s\n", 'b' + mode, T,
           (mode == 0 || mode == 3) ? "one register" : "register x pieces", mode >= 2 ? " (THP)" : "", t1 - t0,
           n / (t1 - t0) / 1e9,
           d2h_gbs(h, d, n));
    if (mode == 0 || mode == 3)
      cudaHostUnregister(h);
    else
      for (int t = 0; t < T; ++t)
        if ((size_t)t * piece < n) cudaHostUnregister((char*)h + t * piece);
    free(h);
  }
  return 0;
}
