// Probe: why do CUDA events around a kernel read long while a copy engine streams over PCIe
// ?  Times the same kernels by events (on the launching stream) and by the device
// clock (%globaltimer written by the kernel), idle / during a 1 GiB D2H / during a 1 GiB H2D, for:
//   ev-ev      two events back to back (no kernel)
//   spin-dev   a 50 us spin kernel that writes its stamps to DEVICE memory
//   spin-host  the same kernel writing its stamps to MAPPED PINNED host memory
//   spin-none  the same kernel, no memory writes at all
//   read-dev   a memory-bound kernel (reads 512 MiB, writes 8 B to device memory)
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/evp tools/event_probe.cu
#include <cstdint>
#include <cstdio>
#include <algorithm>
#include <vector>
#include <cuda_runtime.h>

#define CK(x)                                                                    \
  do {                                                                           \
    cudaError_t e_ = (x);                                                        \
    if (e_ != cudaSuccess) {                                                     \
      printf("FAIL %s: %s\n", #x, cudaGetErrorString(e_));                       \
      return 1;                                                                  \
    }                                                                            \
  } while (0)

__device__ __forceinline__ uint64_t gt() {
  uint64_t a;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(a));
  return a;
}

__global__ void spin(uint64_t ns, uint64_t* t, int write) {
  const uint64_t a = gt();
  uint64_t b;
  do { b = gt(); } while (b - a < ns);
  if (write && threadIdx.x == 0 && blockIdx.x == 0) {
    t[0] = a;
    t[1] = b;
  }
}

__global__ void readk(const uint4* __restrict__ p, uint64_t n16, uint64_t* t) {
  const uint64_t a = gt();
  uint32_t acc = 0;
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n16; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint4 v = __ldcs(p + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x12345678u) t[2] = acc;
  __shared__ uint64_t last;
  __syncthreads();
  if (threadIdx.x == 0) {
    atomicMin(reinterpret_cast<unsigned long long*>(t), (unsigned long long)a);
    last = gt();
    atomicMax(reinterpret_cast<unsigned long long*>(t + 1), (unsigned long long)last);
  }
}

int main() {
  cudaStream_t st, cp;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&cp, cudaStreamNonBlocking));
  uint64_t *th, *td;
  CK(cudaHostAlloc(&th, 64, cudaHostAllocMapped));
  CK(cudaMalloc(&td, 64));
  const size_t big = size_t(1) << 30;
  void *dsrc, *hbuf;
  CK(cudaMalloc(&dsrc, big));
  CK(cudaMemset(dsrc, 1, big));
  CK(cudaHostAlloc(&hbuf, big, 0));
  cudaEvent_t e[3];
  for (auto& x : e) CK(cudaEventCreate(&x));
  const char* bg_names[3] = {"idle", "d2h", "h2d"};
  const char* k_names[5] = {"ev-ev", "spin-dev", "spin-host", "spin-none", "read-dev"};
  for (int bg = 0; bg < 3; bg++) {
    for (int k = 0; k < 5; k++) {
      std::vector<double> evs, devs, tails;
      for (int rep = 0; rep < 7; rep++) {
        CK(cudaDeviceSynchronize());
        CK(cudaMemset(td, 0, 64));
        if (k == 4) {
          uint64_t init[2] = {~0ull, 0};
          CK(cudaMemcpy(td, init, 16, cudaMemcpyHostToDevice));
        }
        if (bg == 1) CK(cudaMemcpyAsync(hbuf, dsrc, big, cudaMemcpyDeviceToHost, cp));
        if (bg == 2) CK(cudaMemcpyAsync(dsrc, hbuf, big, cudaMemcpyHostToDevice, cp));
        // let the copy get going, keep the stream busy so the host enqueues ahead
        spin<<<1, 32, 0, st>>>(200000, td + 4, 0);
        CK(cudaEventRecord(e[0], st));
        uint64_t* t = (k == 2) ? th : td;
        if (k == 1 || k == 2) spin<<<1, 32, 0, st>>>(50000, t, 1);
        if (k == 3) spin<<<1, 32, 0, st>>>(50000, t, 0);
        if (k == 4) readk<<<148 * 4, 512, 0, st>>>(static_cast<const uint4*>(dsrc), (big / 2) / 16, td);
        CK(cudaEventRecord(e[1], st));
        CK(cudaEventRecord(e[2], st));
        CK(cudaStreamSynchronize(st));
        float ms = 0, ms2 = 0;
        CK(cudaEventElapsedTime(&ms, e[0], e[1]));
        CK(cudaEventElapsedTime(&ms2, e[1], e[2]));
        uint64_t s[2] = {0, 0};
        if (k == 2) {
          s[0] = th[0];
          s[1] = th[1];
        } else if (k != 0 && k != 3) {
          CK(cudaMemcpy(s, td, 16, cudaMemcpyDeviceToHost));
        }
        evs.push_back(ms * 1e3);
        tails.push_back(ms2 * 1e3);
        devs.push_back(s[1] > s[0] ? (s[1] - s[0]) / 1e3 : 0.0);
        CK(cudaStreamSynchronize(cp));
      }
      std::sort(evs.begin(), evs.end());
      std::sort(devs.begin(), devs.end());
      std::sort(tails.begin(), tails.end());
      printf("{\"bg\": \"%s\", \"kernel\": \"%s\", \"event_us\": %.1f, \"event_us_min\": %.1f, \"event_us_max\": %.1f, "
             "\"device_clock_us\": %.1f, \"next_event_us\": %.1f}\n",
             bg_names[bg], k_names[k], evs[3], evs[0], evs[6], devs[3], tails[3]);
      fflush(stdout);
    }
  }
  return 0;
}
