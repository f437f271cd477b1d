// Microbenchmark: D2H/H2D bandwidth of 64 MiB copies walking a large pinned host
// buffer, for three ways of pinning it: cudaHostAlloc, 4 KiB pages + cudaHostRegister,
// transparent huge pages (madvise) + cudaHostRegister. Not part of the library.
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <sys/mman.h>
#include <cuda_runtime.h>

static double walk(void* host, size_t total, void* dev, size_t piece, bool d2h, cudaStream_t s) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int w = 0; w < 2; ++w) {  // warm-up pass, timed pass
    cudaEventRecord(a, s);
    for (size_t o = 0; o + piece <= total; o += piece) {
      if (d2h)
        cudaMemcpyAsync((char*)host + o, dev, piece, cudaMemcpyDeviceToHost, s);
      else
        cudaMemcpyAsync(dev, (char*)host + o, piece, cudaMemcpyHostToDevice, s);
    }
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
  }
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  return (double)(total / piece * piece) / (ms * 1e-3) / 1e9;
}

int main(int argc, char** argv) {
  const size_t total = (argc > 1 ? strtoull(argv[1], nullptr, 10) : 8) << 30;
  const size_t piece = 64ull << 20;
  void* dev;
  cudaMalloc(&dev, piece);
  cudaMemset(dev, 1, piece);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  FILE* f = fopen("/sys/kernel/mm/transparent_hugepage/enabled", "r");
  char thp[128] = "?";
  if (f) {
    if (!fgets(thp, sizeof thp, f)) thp[0] = 0;
    fclose(f);
  }
  printf("THP: %s", thp);
  for (int mode = 0; mode < 3; ++mode) {
    void* h = nullptr;
    if (mode == 0) {
      if (cudaHostAlloc(&h, total, cudaHostAllocDefault) != cudaSuccess) { printf("alloc fail\n"); continue; }
    } else {
      h = mmap(nullptr, total + (2 << 20), PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
      h = (void*)(((uintptr_t)h + (2 << 20) - 1) & ~(uintptr_t)((2 << 20) - 1));
      if (mode == 2) printf("madvise %d\n", madvise(h, total, MADV_HUGEPAGE));
      memset(h, 0, total);
      cudaError_t e = cudaHostRegister(h, total, cudaHostRegisterDefault);
      if (e != cudaSuccess) { printf("register fail %s\n", cudaGetErrorString(e)); continue; }
    }
    const char* name[] = {"cudaHostAlloc", "4K pages + register", "THP + register"};
    printf("%-22s D2H %.2f GB/s  H2D %.2f GB/s  (%zu GiB, 64 MiB pieces)\n", name[mode],
           walk(h, total, dev, piece, true, s), walk(h, total, dev, piece, false, s), total >> 30);
    if (mode == 0) cudaFreeHost(h); else cudaHostUnregister(h);
  }
  FILE* m = fopen("/proc/meminfo", "r");
  char line[256];
  while (m && fgets(line, sizeof line, m))
    if (strstr(line, "Huge")) printf("%s", line);
  return 0;
}
