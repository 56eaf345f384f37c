// Experiment: is the CUDA-event time of a kernel launched while a copy engine is busy inflated
// by launch latency?  gate(): the stream waits (cuStreamWaitValue32) on a host flag until the
// host has enqueued the whole launch group, then the host releases it.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC gate_probe.cu -o gate_probe.so
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

typedef CUresult (*WaitValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
static WaitValue32 g_wait = nullptr;
static volatile uint32_t* g_flag = nullptr;
static CUdeviceptr g_flag_dev = 0;

extern "C" int gate_init() {
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint("cuStreamWaitValue32", (void**)&g_wait, cudaEnableDefault, &q) != cudaSuccess || !g_wait)
    return 1;
  void* p = nullptr;
  if (cudaHostAlloc(&p, 64, cudaHostAllocMapped) != cudaSuccess) return 2;
  g_flag = static_cast<volatile uint32_t*>(p);
  *g_flag = 0;
  void* d = nullptr;
  if (cudaHostGetDevicePointer(&d, p, 0) != cudaSuccess) return 3;
  g_flag_dev = reinterpret_cast<CUdeviceptr>(d);
  return 0;
}

extern "C" int gate_close(void* stream, uint32_t seq) {
  return g_wait(static_cast<CUstream>(stream), g_flag_dev, seq, CU_STREAM_WAIT_VALUE_GEQ);
}

extern "C" void gate_open(uint32_t seq) {
  __sync_synchronize();
  *g_flag = seq;
  __sync_synchronize();
}

__global__ void tiny_kernel(int* p) {
  if (threadIdx.x == 0 && blockIdx.x == 0) p[0] += 1;
}

extern "C" void tiny(int* p, void* stream) { tiny_kernel<<<1, 32, 0, static_cast<cudaStream_t>(stream)>>>(p); }
