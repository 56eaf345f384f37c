// Experiment: what does a kernel boundary cost while a copy engine streams D2H / H2D over PCIe,
// for plain stream launches vs the same chain captured in a CUDA graph?  Each kernel stamps
// %globaltimer at entry into slot i (device-side, no events), so the spacing between
// consecutive entries is the per-boundary cost.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC launch_probe.cu -o launch_probe.so
#include <cstdint>
#include <cuda_runtime.h>

__global__ void stamp_kernel(unsigned long long* t, int i) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    unsigned long long g;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g));
    t[i] = g;
  }
}

static cudaGraphExec_t g_exec = nullptr;

extern "C" int chain_plain(unsigned long long* t, int n, int blocks, void* stream) {
  auto s = static_cast<cudaStream_t>(stream);
  for (int i = 0; i < n; i++) stamp_kernel<<<blocks, 128, 0, s>>>(t, i);
  return int(cudaGetLastError());
}

extern "C" int chain_graph_build(unsigned long long* t, int n, int blocks, void* stream) {
  auto s = static_cast<cudaStream_t>(stream);
  cudaGraph_t g;
  if (cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal) != cudaSuccess) return 1;
  for (int i = 0; i < n; i++) stamp_kernel<<<blocks, 128, 0, s>>>(t, i);
  if (cudaStreamEndCapture(s, &g) != cudaSuccess) return 2;
  if (g_exec) cudaGraphExecDestroy(g_exec);
  if (cudaGraphInstantiate(&g_exec, g, 0) != cudaSuccess) return 3;
  cudaGraphDestroy(g);
  if (cudaGraphUpload(g_exec, s) != cudaSuccess) return 4;
  return 0;
}

extern "C" int chain_graph_launch(void* stream) {
  return int(cudaGraphLaunch(g_exec, static_cast<cudaStream_t>(stream)));
}

// graph whose kernel-node parameters are rewritten before every launch
static cudaGraphExec_t g_exec2 = nullptr;
static cudaGraphNode_t g_nodes[256];
static size_t g_nn = 0;
static cudaGraph_t g_graph2 = nullptr;

extern "C" int chain_graph2_build(unsigned long long* t, int n, int blocks, void* stream) {
  auto s = static_cast<cudaStream_t>(stream);
  if (cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal) != cudaSuccess) return 1;
  for (int i = 0; i < n; i++) stamp_kernel<<<blocks, 128, 0, s>>>(t, i);
  if (g_graph2) cudaGraphDestroy(g_graph2);
  if (cudaStreamEndCapture(s, &g_graph2) != cudaSuccess) return 2;
  g_nn = 256;
  if (cudaGraphGetNodes(g_graph2, g_nodes, &g_nn) != cudaSuccess) return 3;
  if (g_exec2) cudaGraphExecDestroy(g_exec2);
  if (cudaGraphInstantiate(&g_exec2, g_graph2, 0) != cudaSuccess) return 4;
  if (cudaGraphUpload(g_exec2, s) != cudaSuccess) return 5;
  return 0;
}

// mode 0: set params of every node then launch; mode 1: re-instantiate + upload + launch;
// mode 2: re-instantiate + launch (no explicit upload)
extern "C" int chain_graph2_launch(unsigned long long* t, int mode, void* stream) {
  auto s = static_cast<cudaStream_t>(stream);
  if (mode == 0) {
    for (size_t k = 0; k < g_nn; k++) {
      cudaKernelNodeParams p;
      if (cudaGraphKernelNodeGetParams(g_nodes[k], &p) != cudaSuccess) return 10;
      unsigned long long* tp = t;
      int i = *static_cast<int*>(p.kernelParams[1]);  // keep the node's index, rewrite the pointer
      void* args[2] = {&tp, &i};
      p.kernelParams = args;
      if (cudaGraphExecKernelNodeSetParams(g_exec2, g_nodes[k], &p) != cudaSuccess) return 11;
    }
    return int(cudaGraphLaunch(g_exec2, s));
  }
  cudaGraphExec_t e;
  if (cudaGraphInstantiate(&e, g_graph2, 0) != cudaSuccess) return 12;
  if (mode == 1 && cudaGraphUpload(e, s) != cudaSuccess) return 13;
  int r = int(cudaGraphLaunch(e, s));
  cudaGraphExecDestroy(e);
  return r;
}

// timing events recorded INSIDE a graph (external event-record nodes) around a kernel chain
static cudaGraphExec_t g_exec3 = nullptr;
extern "C" int chain_graph3_build(unsigned long long* t, int n, int blocks, void* ea, void* eb, void* stream) {
  auto s = static_cast<cudaStream_t>(stream);
  cudaGraph_t g;
  if (cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal) != cudaSuccess) return 1;
  if (cudaEventRecordWithFlags(static_cast<cudaEvent_t>(ea), s, cudaEventRecordExternal) != cudaSuccess) return 6;
  for (int i = 0; i < n; i++) stamp_kernel<<<blocks, 128, 0, s>>>(t, i);
  if (cudaEventRecordWithFlags(static_cast<cudaEvent_t>(eb), s, cudaEventRecordExternal) != cudaSuccess) return 7;
  if (cudaStreamEndCapture(s, &g) != cudaSuccess) return 2;
  if (g_exec3) cudaGraphExecDestroy(g_exec3);
  if (cudaGraphInstantiate(&g_exec3, g, 0) != cudaSuccess) return 3;
  cudaGraphDestroy(g);
  if (cudaGraphUpload(g_exec3, s) != cudaSuccess) return 4;
  return 0;
}
extern "C" int chain_graph3_launch(void* stream) { return int(cudaGraphLaunch(g_exec3, static_cast<cudaStream_t>(stream))); }
