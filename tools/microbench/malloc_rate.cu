// Microbenchmark: device allocation rates on B200 — cudaMalloc of one 5 GiB block, of
// 80 blocks of 64 MiB, and cudaMallocAsync from the default pool (first and second use).
// Not part of the library.
#include <chrono>
#include <cstdio>
#include <vector>
#include <cuda_runtime.h>

static double now() { return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count(); }

int main() {
  cudaFree(0);
  const size_t big = 5ull << 30, seg = 64ull << 20;
  const int nseg = (int)(big / seg);
  for (int rep = 0; rep < 2; ++rep) {
    double t0 = now();
    void* p;
    cudaMalloc(&p, big);
    double t1 = now();
    cudaFree(p);
    double t2 = now();
    std::vector<void*> v(nseg);
    for (auto& q : v) cudaMalloc(&q, seg);
    double t3 = now();
    for (auto q : v) cudaFree(q);
    double t4 = now();
    printf("rep %d: cudaMalloc 5 GiB %.1f ms (free %.1f ms); %d x 64 MiB %.1f ms (free %.1f ms)\n", rep, (t1 - t0) * 1e3,
           (t2 - t1) * 1e3, nseg, (t3 - t2) * 1e3, (t4 - t3) * 1e3);
  }
  cudaStream_t s;
  cudaStreamCreate(&s);
  for (int rep = 0; rep < 2; ++rep) {
    double t0 = now();
    std::vector<void*> v(nseg);
    for (auto& q : v) cudaMallocAsync(&q, seg, s);
    cudaStreamSynchronize(s);
    double t1 = now();
    for (auto q : v) cudaFreeAsync(q, s);
    cudaStreamSynchronize(s);
    printf("cudaMallocAsync %d x 64 MiB rep %d: %.1f ms\n", nseg, rep, (t1 - t0) * 1e3);
  }
  return 0;
}
