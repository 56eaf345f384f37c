// Probe: D2H copy-engine rate by source allocation (cudaMalloc / default stream-ordered pool /
// a private cudaMemPoolCreate pool) and destination (cudaHostAlloc flags, offsets inside a
// 512 MiB chunk), 64 MiB per copy, best and median of 7 (the swap-out D2H rate).
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/d2hp tools/d2h_probe.cu
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <vector>
#include <cuda_runtime.h>

#define CK(x)                                                              \
  do {                                                                     \
    cudaError_t e_ = (x);                                                  \
    if (e_ != cudaSuccess) {                                               \
      printf("FAIL %s: %s\n", #x, cudaGetErrorString(e_));                 \
      return 1;                                                            \
    }                                                                      \
  } while (0)

int main() {
  const size_t B = size_t(64) << 20, CH = size_t(512) << 20;
  cudaStream_t st;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  void *s_malloc, *s_default, *s_private;
  CK(cudaMalloc(&s_malloc, B));
  CK(cudaMallocAsync(&s_default, B, st));
  cudaMemPool_t pool;
  cudaMemPoolProps pp = {};
  pp.allocType = cudaMemAllocationTypePinned;
  pp.location.type = cudaMemLocationTypeDevice;
  pp.location.id = 0;
  CK(cudaMemPoolCreate(&pool, &pp));
  CK(cudaMallocFromPoolAsync(&s_private, B, pool, st));
  CK(cudaStreamSynchronize(st));
  void *h_default, *h_mapped, *h_wc;
  CK(cudaHostAlloc(&h_default, CH, cudaHostAllocDefault));
  CK(cudaHostAlloc(&h_mapped, CH, cudaHostAllocPortable | cudaHostAllocMapped));
  CK(cudaHostAlloc(&h_wc, CH, cudaHostAllocPortable | cudaHostAllocMapped | cudaHostAllocWriteCombined));
  const char* sn[3] = {"cudaMalloc", "default_pool", "private_pool"};
  void* srcs[3] = {s_malloc, s_default, s_private};
  const char* dn[3] = {"hostalloc_default", "portable_mapped", "portable_mapped_wc"};
  void* dsts[3] = {h_default, h_mapped, h_wc};
  size_t offs[4] = {0, 256, 4096 + 256, size_t(200) << 20};
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  for (int si = 0; si < 3; si++)
    for (int di = 0; di < 3; di++)
      for (size_t off : offs) {
        std::vector<float> t;
        for (int r = 0; r < 7; r++) {
          CK(cudaEventRecord(a, st));
          CK(cudaMemcpyAsync(static_cast<char*>(dsts[di]) + off, srcs[si], B, cudaMemcpyDeviceToHost, st));
          CK(cudaEventRecord(b, st));
          CK(cudaEventSynchronize(b));
          float ms;
          CK(cudaEventElapsedTime(&ms, a, b));
          t.push_back(ms);
        }
        std::sort(t.begin(), t.end());
        printf("{\"src\": \"%s\", \"dst\": \"%s\", \"offset\": %zu, \"best_GBps\": %.2f, \"median_GBps\": %.2f}\n",
               sn[si], dn[di], off, B / (t[0] * 1e-3) / 1e9, B / (t[3] * 1e-3) / 1e9);
      }
  // H2D too, for completeness
  for (int di = 0; di < 3; di++) {
    std::vector<float> t;
    for (int r = 0; r < 7; r++) {
      CK(cudaEventRecord(a, st));
      CK(cudaMemcpyAsync(s_private, dsts[di], B, cudaMemcpyHostToDevice, st));
      CK(cudaEventRecord(b, st));
      CK(cudaEventSynchronize(b));
      float ms;
      CK(cudaEventElapsedTime(&ms, a, b));
      t.push_back(ms);
    }
    std::sort(t.begin(), t.end());
    printf("{\"h2d_from\": \"%s\", \"best_GBps\": %.2f, \"median_GBps\": %.2f}\n", dn[di], B / (t[0] * 1e-3) / 1e9,
           B / (t[3] * 1e-3) / 1e9);
  }
  return 0;
}
