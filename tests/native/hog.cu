// Test helper (not product code): a kernel that occupies whole SMs for a while, to check that
// the persistent ZVC compress makes progress when it is not alone on the GPU
// (tests/test_gpu_concurrency.py).  nvcc -shared -Xcompiler -fPIC -gencode
// arch=compute_100a,code=sm_100a hog.cu -o libhog.so
#include <cstdint>
#include <cuda_runtime.h>

__global__ void hog_kernel(uint64_t ns, int* sink) {
  extern __shared__ int smem[];
  uint64_t a, b;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(a));
  do {
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(b));
  } while (b - a < ns);
  if (threadIdx.x == 0) smem[0] = int(b - a);
  __syncthreads();
  if (threadIdx.x == 0 && smem[0] == 0x7fffffff) *sink = 1;
}

// `ctas` CTAs of 1024 threads with `smem_bytes` of shared memory each (>= 120 KiB keeps one CTA
// per SM), each spinning for `ns` nanoseconds
extern "C" int hog_launch(int ctas, int smem_bytes, uint64_t ns, int* sink, void* stream) {
  cudaFuncSetAttribute(hog_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
  hog_kernel<<<ctas, 1024, smem_bytes, (cudaStream_t)stream>>>(ns, sink);
  return (int)cudaGetLastError();
}
