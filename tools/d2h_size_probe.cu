// Probe: D2H copy-engine rate of ONE copy by size (64 MiB .. 2 GiB), source cudaMalloc, destination
// cudaHostAlloc(Portable | Mapped) — in-step copies of 400-800 MB ran at 52.3 GB/s while 64-256 MiB
// copies run at 56-57.  nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/d2hs tools/d2h_size_probe.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

int main() {
  const size_t maxb = size_t(2) << 30;
  void *dev, *host;
  cudaMalloc(&dev, maxb);
  cudaMemset(dev, 1, maxb);
  cudaHostAlloc(&host, maxb, cudaHostAllocPortable | cudaHostAllocMapped);
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int rep = 0; rep < 2; rep++)
    for (size_t mib : {16, 64, 128, 256, 512, 784, 1024, 2048}) {
      for (int dir = 0; dir < 2; dir++) {
        const size_t bytes = mib << 20;
        float best = 1e9;
        for (int r = 0; r < 3; r++) {
          cudaEventRecord(a, st);
          if (dir == 0) cudaMemcpyAsync(host, dev, bytes, cudaMemcpyDeviceToHost, st);
          else cudaMemcpyAsync(dev, host, bytes, cudaMemcpyHostToDevice, st);
          cudaEventRecord(b, st);
          cudaEventSynchronize(b);
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          best = ms < best ? ms : best;
        }
        printf("{\"rep\": %d, \"dir\": \"%s\", \"MiB\": %zu, \"GBps\": %.2f}\n", rep, dir ? "h2d" : "d2h", mib,
               bytes / (best * 1e-3) / 1e9);
      }
    }
  return 0;
}
