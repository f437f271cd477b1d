// Microbenchmark: D2H/H2D bandwidth of 64 MiB copies walking a large pinned host
// buffer, for three ways of pinning it: cudaHostAlloc, 4 KiB pages + cudaHostRegister,
// transparent huge pages (madvise) + cudaHostRegister. Not part of the library.
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <sys/mman.h>
#include <cuda_runtime.h>

__global__ void hbm_copy(const uint4* a, uint4* b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}

static double walk(void* host, size_t total, void* dev, size_t piece, bool d2h, cudaStream_t s, size_t shift = 0,
                   size_t step = 0, cudaStream_t busy = nullptr, uint4* hb = nullptr, bool coalign = false, bool split = false) {
  step = step ? step : piece;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int w = 0; w < 2; ++w) {  // warm-up pass, timed pass
    cudaEventRecord(a, s);
    for (size_t o = shift; o + piece <= total; o += step) {
      if (busy) hbm_copy<<<148 * 4, 512, 0, busy>>>(hb, hb + (32 << 20) / 16, (32 << 20) / 16);  // 64 MiB of HBM traffic
      char* src = (char*)dev + (coalign ? (((uintptr_t)host + o) & 4095) : 0);
      if (split && d2h) {  // head to the next 4 KiB boundary, aligned middle, tail
        const uintptr_t d0 = (uintptr_t)host + o, d1 = d0 + piece;
        const uintptr_t a0 = (d0 + 4095) & ~(uintptr_t)4095, a1 = d1 & ~(uintptr_t)4095;
        if (a0 > d0) cudaMemcpyAsync((void*)d0, src, a0 - d0, cudaMemcpyDeviceToHost, s);
        cudaMemcpyAsync((void*)a0, src + (a0 - d0), a1 - a0, cudaMemcpyDeviceToHost, s);
        if (d1 > a1) cudaMemcpyAsync((void*)a1, src + (a1 - d0), d1 - a1, cudaMemcpyDeviceToHost, s);
        continue;
      }
      if (d2h)
        cudaMemcpyAsync((char*)host + o, src, piece, cudaMemcpyDeviceToHost, s);
      else
        cudaMemcpyAsync(dev, (char*)host + o, piece, cudaMemcpyHostToDevice, s);
    }
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
  }
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  size_t moved = 0;
  for (size_t o = shift; o + piece <= total; o += step) moved += piece;
  return (double)moved / (ms * 1e-3) / 1e9;
}

int main(int argc, char** argv) {
  const size_t total = (argc > 1 ? strtoull(argv[1], nullptr, 10) : 8) << 30;
  const size_t piece = 64ull << 20;
  void* dev;
  cudaMalloc(&dev, piece + 8192);
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
    if (mode == 0) {
      // the checkpoint pipeline's shapes: destinations 256-B aligned (odd buffers), pieces
      // of 64 MiB + 37 KiB, and an HBM-heavy kernel on another stream per piece
      cudaStream_t busy;
      cudaStreamCreateWithFlags(&busy, cudaStreamNonBlocking);
      uint4* hb;
      cudaMalloc(&hb, 64 << 20);
      printf("  dest +256 B           D2H %.2f GB/s  H2D %.2f GB/s\n", walk(h, total, dev, piece, true, s, 256),
             walk(h, total, dev, piece, false, s, 256));
      printf("  odd piece, +256 step  D2H %.2f GB/s\n", walk(h, total, dev, piece - 37 * 1024 - 256, true, s, 0,
                                                          piece - 37 * 1024));
      printf("  odd piece, co-aligned D2H %.2f GB/s\n", walk(h, total, dev, piece - 37 * 1024 - 256, true, s, 0,
                                                          piece - 37 * 1024, nullptr, nullptr, true));
      printf("  odd piece, split head/mid/tail D2H %.2f GB/s\n", walk(h, total, dev, piece - 37 * 1024 - 256, true, s, 0,
                                                          piece - 37 * 1024 - 256, nullptr, nullptr, false, true));
      printf("  odd piece, contiguous D2H %.2f GB/s\n", walk(h, total, dev, piece - 37 * 1024 - 256, true, s, 0,
                                                          piece - 37 * 1024 - 256));
      printf("  aligned starts, odd size D2H %.2f GB/s\n", walk(h, total, dev, piece - 37 * 1024 - 256, true, s, 0,
                                                          piece));
      printf("  drifting starts, 64 MiB size D2H %.2f GB/s\n", walk(h, total, dev, piece - 40 * 1024, true, s, 0,
                                                          piece - 37 * 1024 - 256));
      printf("  with HBM kernel       D2H %.2f GB/s  H2D %.2f GB/s\n", walk(h, total, dev, piece, true, s, 0, 0, busy, hb),
             walk(h, total, dev, piece, false, s, 0, 0, busy, hb));
      cudaFreeHost(h);
    } else {
      cudaHostUnregister(h);
    }
  }
  FILE* m = fopen("/proc/meminfo", "r");
  char line[256];
  while (m && fgets(line, sizeof line, m))
    if (strstr(line, "Huge")) printf("%s", line);
  return 0;
}
