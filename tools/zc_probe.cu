// Experiment: SM-driven copies between device memory and mapped pinned host memory (no copy
// engine), to compare link throughput and interference with the copy-engine path.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC zc_probe.cu -o zc_probe.so
#include <cstdint>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(256) d2h_kernel(const uint4* __restrict__ src, uint4* dst, uint64_t n16) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x * 4;
  for (uint64_t i = (uint64_t(blockIdx.x) * blockDim.x) * 4 + threadIdx.x; i < n16; i += stride) {
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; u++) {
      const uint64_t j = i + uint64_t(u) * blockDim.x;
      if (j < n16) v[u] = __ldcs(src + j);
    }
#pragma unroll
    for (int u = 0; u < 4; u++) {
      const uint64_t j = i + uint64_t(u) * blockDim.x;
      if (j < n16) __stcs(dst + j, v[u]);
    }
  }
}

__global__ void __launch_bounds__(256) h2d_kernel(const uint4* src, uint4* __restrict__ dst, uint64_t n16) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x * 8;
  for (uint64_t i = (uint64_t(blockIdx.x) * blockDim.x) * 8 + threadIdx.x; i < n16; i += stride) {
    uint4 v[8];
#pragma unroll
    for (int u = 0; u < 8; u++) {
      const uint64_t j = i + uint64_t(u) * blockDim.x;
      if (j < n16) v[u] = __ldcv(src + j);
    }
#pragma unroll
    for (int u = 0; u < 8; u++) {
      const uint64_t j = i + uint64_t(u) * blockDim.x;
      if (j < n16) __stcs(dst + j, v[u]);
    }
  }
}

extern "C" int zc_d2h(const void* src, void* host, uint64_t bytes, int ctas, void* stream) {
  void* dptr = nullptr;
  if (cudaHostGetDevicePointer(&dptr, host, 0) != cudaSuccess) return 1;
  d2h_kernel<<<ctas, 256, 0, (cudaStream_t)stream>>>((const uint4*)src, (uint4*)dptr, bytes / 16);
  return cudaGetLastError();
}

extern "C" int zc_h2d(const void* host, void* dst, uint64_t bytes, int ctas, void* stream) {
  void* dptr = nullptr;
  if (cudaHostGetDevicePointer(&dptr, const_cast<void*>(host), 0) != cudaSuccess) return 1;
  h2d_kernel<<<ctas, 256, 0, (cudaStream_t)stream>>>((const uint4*)dptr, (uint4*)dst, bytes / 16);
  return cudaGetLastError();
}
