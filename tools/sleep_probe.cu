// Probe: how long does __nanosleep(t) actually suspend a warp on B200, and how often does
// mbarrier.try_wait (with and without a suspend-time hint) return on a phase that never
// completes?  (The persistent compress's polling loops were ~22 % of its issued instructions in
// the round-2 ncu source view.)  nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/slp tools/sleep_probe.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t gt() {
  uint64_t a;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(a));
  return a;
}

__global__ void sleep_k(uint32_t ns, int iters, uint64_t* out) {
  const uint64_t a = gt();
  for (int i = 0; i < iters; i++) __nanosleep(ns);
  const uint64_t b = gt();
  if (threadIdx.x == 0) out[blockIdx.x] = b - a;
}

__global__ void trywait_k(uint32_t hint_ns, int iters, uint64_t* out) {
  __shared__ __align__(8) uint64_t bar;
  if (threadIdx.x == 0) {
    const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(&bar));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(a));
  }
  __syncthreads();
  const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(&bar));
  const uint64_t t0 = gt();
  uint32_t done = 0;
  for (int i = 0; i < iters; i++) {
    uint32_t ok;
    if (hint_ns)
      asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0, %2;\nselp.u32 %0, 1, 0, p;\n}"
                   : "=r"(ok) : "r"(a), "r"(hint_ns) : "memory");
    else
      asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\nselp.u32 %0, 1, 0, p;\n}"
                   : "=r"(ok) : "r"(a) : "memory");
    done += ok;
  }
  const uint64_t t1 = gt();
  if (threadIdx.x == 0) out[blockIdx.x] = (t1 - t0) | (uint64_t(done) << 48);
}

int main() {
  uint64_t* d;
  cudaMalloc(&d, 4096 * 8);
  uint64_t h[4096];
  const int iters = 200;
  for (int warps : {1, 8}) {
    for (uint32_t ns : {0u, 32u, 64u, 256u, 1000u, 10000u}) {
      sleep_k<<<148, 32 * warps>>>(ns, iters, d);
      cudaDeviceSynchronize();
      cudaMemcpy(h, d, 148 * 8, cudaMemcpyDeviceToHost);
      double m = 0;
      for (int i = 0; i < 148; i++) m += h[i];
      printf("{\"probe\": \"nanosleep\", \"warps_per_cta\": %d, \"ns\": %u, \"actual_ns_per_call\": %.1f}\n", warps, ns,
             m / 148 / iters);
    }
  }
  for (uint32_t hint : {0u, 1000u, 100000u}) {
    trywait_k<<<148, 32>>>(hint, iters, d);
    cudaDeviceSynchronize();
    cudaMemcpy(h, d, 148 * 8, cudaMemcpyDeviceToHost);
    double m = 0;
    for (int i = 0; i < 148; i++) m += h[i] & ((1ull << 48) - 1);
    printf("{\"probe\": \"try_wait(never completes)\", \"hint_ns\": %u, \"actual_ns_per_call\": %.1f, \"completed\": %llu}\n",
           hint, m / 148 / iters, (unsigned long long)(h[0] >> 48));
  }
  return 0;
}
