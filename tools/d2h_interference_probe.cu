// Probe: does other GPU work slow a D2H copy on this box?  In the swap steps
// the D2H copies move 51-57 GB/s against 57.2 for one copy alone.  A 2 GiB device -> pinned copy
// runs while another stream launches, every `gap` microseconds of host time, either nothing, a
// 1-thread kernel storing 8 bytes to HOST-mapped memory (like the probe's counts and the
// compress's progress words), the same kernel storing to DEVICE memory, a timing-event pair, or
// an HBM-heavy kernel (a 256 MiB device-to-device copy kernel: compress-like traffic).
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/dip tools/d2h_interference_probe.cu
#include <cstdio>
#include <cstdint>
#include <chrono>
#include <thread>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("FAIL %s: %s\n", #x, cudaGetErrorString(e_)); return 1; } } while (0)

__global__ void poke(uint64_t* p) { *p = 1; }
__global__ void dcopy(const uint4* __restrict__ a, uint4* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * size_t(blockDim.x) + threadIdx.x; i < n; i += size_t(gridDim.x) * blockDim.x) b[i] = a[i];
}

int main() {
  const size_t big = size_t(2) << 30, hb = size_t(256) << 20;
  void *dsrc, *hdst, *ha, *hbuf;
  CK(cudaMalloc(&dsrc, big));
  CK(cudaHostAlloc(&hdst, big, 0));
  CK(cudaMalloc(&ha, hb));
  CK(cudaMalloc(&hbuf, hb));
  uint64_t *hmap, *dword;
  CK(cudaHostAlloc(&hmap, 64, cudaHostAllocMapped));
  CK(cudaMalloc(&dword, 64));
  cudaStream_t cp, ks;
  CK(cudaStreamCreateWithFlags(&cp, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&ks, cudaStreamNonBlocking));
  cudaEvent_t a, b, e0, e1;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  const char* names[5] = {"nothing", "kernel_store_host", "kernel_store_device", "timing_event_pair", "hbm_copy_kernel_256MiB"};
  for (int gap_us : {100, 25}) {
    for (int mode = 0; mode < 5; mode++) {
      float best = 1e9;
      int launches = 0;
      for (int rep = 0; rep < 3; rep++) {
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(a, cp));
        CK(cudaMemcpyAsync(hdst, dsrc, big, cudaMemcpyDeviceToHost, cp));
        CK(cudaEventRecord(b, cp));
        launches = 0;
        while (cudaEventQuery(b) == cudaErrorNotReady) {
          if (mode == 1) poke<<<1, 1, 0, ks>>>(hmap);
          if (mode == 2) poke<<<1, 1, 0, ks>>>(dword);
          if (mode == 3) { CK(cudaEventRecord(e0, ks)); CK(cudaEventRecord(e1, ks)); }
          if (mode == 4) dcopy<<<592, 512, 0, ks>>>((const uint4*)ha, (uint4*)hbuf, hb / 16);
          launches += mode != 0;
          std::this_thread::sleep_for(std::chrono::microseconds(mode == 4 ? gap_us * 4 : gap_us));
        }
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, a, b));
        if (ms < best) best = ms;
      }
      printf("{\"gap_us\": %d, \"beside_d2h\": \"%s\", \"launches\": %d, \"d2h_GBps\": %.2f}\n", gap_us, names[mode], launches,
             big / (best * 1e-3) / 1e9);
      fflush(stdout);
    }
  }
  return 0;
}
