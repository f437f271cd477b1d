// Diagnostic: which CUDA graph exec update does the runtime accept for a kernel node
// with > 48 KB dynamic shared memory and a by-value struct parameter. Not part of the library.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

struct P { const uint8_t* a; uint64_t b[20]; int* sink; };

__global__ void k(const P p) {
  extern __shared__ uint8_t sm[];
  if (threadIdx.x == 0 && p.sink) sm[0] = 1, p.sink[blockIdx.x] = (int)p.b[0];
}

#define CK(x) do { cudaError_t e = (x); printf("%-60s %s\n", #x, cudaGetErrorString(e)); } while (0)

int main() {
  const size_t smem = 217 * 1024;
  CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int* sink;
  cudaMalloc(&sink, 4096);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaEvent_t a, b, a2, b2;
  cudaEventCreate(&a); cudaEventCreate(&b); cudaEventCreate(&a2); cudaEventCreate(&b2);
  P p = {};
  p.sink = sink;
  p.b[0] = 7;
  void* args[] = {&p};
  cudaKernelNodeParams kp = {};
  kp.func = (void*)k;
  kp.gridDim = dim3(148);
  kp.blockDim = dim3(320);
  kp.sharedMemBytes = (unsigned)smem;
  kp.kernelParams = args;
  cudaGraph_t g;
  cudaGraphNode_t na, nk, nb;
  CK(cudaGraphCreate(&g, 0));
  CK(cudaGraphAddEventRecordNode(&na, g, nullptr, 0, a));
  CK(cudaGraphAddKernelNode(&nk, g, &na, 1, &kp));
  CK(cudaGraphAddEventRecordNode(&nb, g, &nk, 1, b));
  cudaGraphExec_t ge;
  CK(cudaGraphInstantiate(&ge, g, 0));
  CK(cudaGraphLaunch(ge, s));
  CK(cudaStreamSynchronize(s));
  p.b[0] = 9;
  CK(cudaGraphExecKernelNodeSetParams(ge, nk, &kp));
  CK(cudaGraphExecEventRecordNodeSetEvent(ge, na, a2));
  CK(cudaGraphExecEventRecordNodeSetEvent(ge, nb, b2));
  CK(cudaGraphLaunch(ge, s));
  CK(cudaStreamSynchronize(s));
  int h = 0;
  cudaMemcpy(&h, sink, 4, cudaMemcpyDeviceToHost);
  printf("sink %d (want 9)\n", h);
  // smaller grid through the update
  kp.gridDim = dim3(77);
  p.b[0] = 11;
  CK(cudaGraphExecKernelNodeSetParams(ge, nk, &kp));
  CK(cudaGraphLaunch(ge, s));
  CK(cudaStreamSynchronize(s));
  // set the attribute on the node instead
  cudaKernelNodeAttrValue v = {};
  CK(cudaGraphKernelNodeGetAttribute(nk, cudaKernelNodeAttributePriority, &v));
  // generic update path (CUDA 12.2+)
  cudaGraphNodeParams np = {};
  np.type = cudaGraphNodeTypeKernel;
  np.kernel.func = (void*)k;
  np.kernel.gridDim = dim3(148);
  np.kernel.blockDim = dim3(320);
  np.kernel.sharedMemBytes = (unsigned)smem;
  np.kernel.kernelParams = args;
  p.b[0] = 13;
  CK(cudaGraphExecNodeSetParams(ge, nk, &np));
  CK(cudaGraphLaunch(ge, s));
  CK(cudaStreamSynchronize(s));
  cudaMemcpy(&h, sink, 4, cudaMemcpyDeviceToHost);
  printf("sink %d (want 13)\n", h);
  // in-flight update: launch, update, launch, no sync in between
  for (int i = 0; i < 3; ++i) {
    p.b[0] = 20 + i;
    CK(cudaGraphExecKernelNodeSetParams(ge, nk, &kp));
    CK(cudaGraphExecEventRecordNodeSetEvent(ge, na, (i & 1) ? a : a2));
    CK(cudaGraphExecEventRecordNodeSetEvent(ge, nb, (i & 1) ? b : b2));
    CK(cudaGraphLaunch(ge, s));
  }
  CK(cudaStreamSynchronize(s));
  cudaMemcpy(&h, sink, 4, cudaMemcpyDeviceToHost);
  printf("sink %d (want 22)\n", h);
  return 0;
}
