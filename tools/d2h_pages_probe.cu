// Probe: does the D2H copy rate depend on how much distinct host memory the copies land in (IOMMU /
// IOTLB reach in the VM) and on how that memory was pinned?  64 MiB copies into successive offsets
// of a 2 GiB buffer (cold pages) vs 32 repeats into the same 64 MiB (warm), for memory from
// cudaHostAlloc, and malloc'd / mmap'd-with-MADV_HUGEPAGE memory registered with cudaHostRegister.
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/d2hpg tools/d2h_pages_probe.cu
#include <sys/mman.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <cuda_runtime.h>

static double run(void* host, size_t span, size_t chunk, bool same, cudaStream_t st, void* dev) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int n = int(span / chunk);
  cudaEventRecord(a, st);
  for (int i = 0; i < n; i++)
    cudaMemcpyAsync(static_cast<char*>(host) + (same ? 0 : size_t(i) * chunk), dev, chunk, cudaMemcpyDeviceToHost, st);
  cudaEventRecord(b, st);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  return double(span) / (ms * 1e-3) / 1e9;
}

int main() {
  const size_t span = size_t(2) << 30, chunk = size_t(64) << 20;
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  void* dev;
  cudaMalloc(&dev, chunk);
  cudaMemset(dev, 1, chunk);
  struct Src { const char* name; void* p; };
  std::vector<Src> srcs;
  void* h1 = nullptr;
  if (cudaHostAlloc(&h1, span, cudaHostAllocPortable | cudaHostAllocMapped) != cudaSuccess) {
    printf("cudaHostAlloc failed\n");
    return 1;
  }
  srcs.push_back({"cudaHostAlloc", h1});
  printf("allocated\n");
  fflush(stdout);
  void* h2 = aligned_alloc(4096, span);
  memset(h2, 0, span);
  if (cudaHostRegister(h2, span, cudaHostRegisterPortable) == cudaSuccess) srcs.push_back({"malloc+register", h2});
  else printf("register(malloc) failed: %s\n", cudaGetErrorString(cudaGetLastError()));
  void* h3 = mmap(nullptr, span, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  int adv = madvise(h3, span, MADV_HUGEPAGE);
  memset(h3, 0, span);
  cudaError_t e = cudaHostRegister(h3, span, cudaHostRegisterPortable);
  if (e == cudaSuccess) srcs.push_back({adv == 0 ? "mmap+THP+register" : "mmap(THP failed)+register", h3});
  else printf("register(mmap) failed: %s\n", cudaGetErrorString(e));
  fflush(stdout);
  for (int rep = 0; rep < 2; rep++)
    for (auto& s : srcs) {
      const double cold = run(s.p, span, chunk, false, st, dev);
      const double warm = run(s.p, span, chunk, true, st, dev);
      printf("{\"host\": \"%s\", \"rep\": %d, \"successive_64MiB_GBps\": %.2f, \"same_64MiB_GBps\": %.2f}\n", s.name, rep,
             cold, warm);
      fflush(stdout);
    }
  return 0;
}
