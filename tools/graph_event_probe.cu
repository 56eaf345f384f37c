// Probe: can timing events be recorded by event-record nodes INSIDE a CUDA graph, and do such
// events bracket the kernel more tightly than events recorded on the stream around the graph
// launch while a D2H copy streams over PCIe?
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/gep tools/graph_event_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("FAIL %s: %s\n", #x, cudaGetErrorString(e_)); return 1; } } while (0)

__global__ void spin(uint64_t ns, uint64_t* t) {
  uint64_t a, b;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(a));
  do { asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(b)); } while (b - a < ns);
  if (threadIdx.x == 0 && blockIdx.x == 0) { t[0] = a; t[1] = b; }
}

static void* spin_args[2];

int main() {
  cudaStream_t st, cp, cap;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&cp, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
  uint64_t* t;
  CK(cudaHostAlloc(&t, 16, cudaHostAllocMapped));
  const size_t big = size_t(1) << 30;
  void *dsrc, *hdst;
  CK(cudaMalloc(&dsrc, big));
  CK(cudaHostAlloc(&hdst, big, 0));
  cudaEvent_t ea, eb, ga, gb;
  CK(cudaEventCreate(&ea)); CK(cudaEventCreate(&eb)); CK(cudaEventCreate(&ga)); CK(cudaEventCreate(&gb));
  // graph: event node (ga) -> kernel (captured) -> event node (gb)
  uint64_t ns = 50000;
  CK(cudaStreamBeginCapture(cap, cudaStreamCaptureModeRelaxed));
  spin<<<1, 32, 0, cap>>>(ns, t);
  cudaGraph_t g;
  CK(cudaStreamEndCapture(cap, &g));
  size_t nroot = 0;
  CK(cudaGraphGetRootNodes(g, nullptr, &nroot));
  cudaGraphNode_t roots[8];
  CK(cudaGraphGetRootNodes(g, roots, &nroot));
  cudaGraphNode_t na, nb;
  CK(cudaGraphAddEventRecordNode(&na, g, nullptr, 0, ga));
  for (size_t i = 0; i < nroot; i++) CK(cudaGraphAddDependencies(g, &na, &roots[i], 1));
  CK(cudaGraphAddEventRecordNode(&nb, g, roots, nroot, gb));
  cudaGraphExec_t ex;
  CK(cudaGraphInstantiate(&ex, g, 0));
  CK(cudaGraphUpload(ex, st));
  for (int mode = 0; mode < 2; mode++) {
    for (int rep = 0; rep < 4; rep++) {
      if (mode) CK(cudaMemcpyAsync(hdst, dsrc, big, cudaMemcpyDeviceToHost, cp));
      CK(cudaEventRecord(ea, st));
      CK(cudaGraphLaunch(ex, st));
      CK(cudaEventRecord(eb, st));
      CK(cudaStreamSynchronize(st));
      float outer = 0, inner = 0;
      CK(cudaEventElapsedTime(&outer, ea, eb));
      CK(cudaEventElapsedTime(&inner, ga, gb));
      printf("%s rep %d: kernel (globaltimer) %.1f us | events around launch %.1f us | event nodes in graph %.1f us\n",
             mode ? "during 1 GiB D2H" : "idle", rep, (t[1] - t[0]) / 1000.0, outer * 1000, inner * 1000);
      CK(cudaStreamSynchronize(cp));
    }
  }
  // swap the recorded events through cudaGraphExecUpdate (what run_group would do per call)
  cudaEvent_t ga2, gb2;
  CK(cudaEventCreate(&ga2)); CK(cudaEventCreate(&gb2));
  CK(cudaGraphEventRecordNodeSetEvent(na, ga2));
  CK(cudaGraphEventRecordNodeSetEvent(nb, gb2));
  cudaGraphExecUpdateResultInfo info;
  CK(cudaGraphExecUpdate(ex, g, &info));
  CK(cudaGraphLaunch(ex, st));
  CK(cudaStreamSynchronize(st));
  float inner = 0;
  CK(cudaEventElapsedTime(&inner, ga2, gb2));
  printf("after ExecUpdate with new events: %.1f us\n", inner * 1000);
  printf("OK\n");
  return 0;
}
