// Probe: what does each stream operation between two kernels cost while a copy engine streams
// over PCIe?  Two 1-thread stamp kernels read %globaltimer; the gap between the
// first one's end stamp and the second one's start stamp is the stream time of what sits between
// them: nothing, a timing event record, a disable-timing event record, a wait on a completed
// event, or the same inside a graph (event-record nodes, graph kernel boundary).
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/egp tools/event_gap_probe.cu
#include <cstdio>
#include <cstdint>
#include <algorithm>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("FAIL %s: %s\n", #x, cudaGetErrorString(e_)); return 1; } } while (0)

__global__ void stamp(uint64_t* t) {
  uint64_t a;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(a));
  *t = a;
}

// spins ns nanoseconds; stamps its start and end into device memory
__global__ void spin(uint64_t ns, uint64_t* t) {
  uint64_t a, b;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(a));
  do { asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(b)); } while (b - a < ns);
  t[0] = a;
  t[1] = b;
}

int main() {
  cudaStream_t st, cp, cap;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&cp, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
  uint64_t* t;
  CK(cudaHostAlloc(&t, 64, cudaHostAllocMapped));
  uint64_t* td;
  CK(cudaMalloc(&td, 64));
  const size_t big = size_t(1) << 30;
  void *dsrc, *hdst, *hsrc, *ddst;
  CK(cudaMalloc(&dsrc, big));
  CK(cudaMalloc(&ddst, big));
  CK(cudaHostAlloc(&hdst, big, 0));
  CK(cudaHostAlloc(&hsrc, big, 0));
  cudaEvent_t et, ent, done, ga, gb;
  CK(cudaEventCreate(&et));
  CK(cudaEventCreateWithFlags(&ent, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&done, cudaEventDisableTiming));
  CK(cudaEventCreate(&ga));
  CK(cudaEventCreate(&gb));
  CK(cudaEventRecord(done, cp));
  CK(cudaStreamSynchronize(cp));

  // graph: stamp -> [event node ga] -> stamp -> [event node gb] -> stamp (device memory stamps)
  cudaGraph_t g;
  CK(cudaGraphCreate(&g, 0));
  cudaKernelNodeParams kp = {};
  void* args0[1];
  uint64_t* p0 = td;
  uint64_t* p1 = td + 1;
  uint64_t* p2 = td + 2;
  args0[0] = &p0;
  kp.func = (void*)stamp;
  kp.gridDim = dim3(1);
  kp.blockDim = dim3(1);
  kp.kernelParams = args0;
  cudaGraphNode_t k0, k1, k2, na, nb;
  CK(cudaGraphAddKernelNode(&k0, g, nullptr, 0, &kp));
  CK(cudaGraphAddEventRecordNode(&na, g, &k0, 1, ga));
  void* args1[1] = {&p1};
  kp.kernelParams = args1;
  CK(cudaGraphAddKernelNode(&k1, g, &na, 1, &kp));
  CK(cudaGraphAddEventRecordNode(&nb, g, &k1, 1, gb));
  void* args2[1] = {&p2};
  kp.kernelParams = args2;
  CK(cudaGraphAddKernelNode(&k2, g, &nb, 1, &kp));
  cudaGraphExec_t ex;
  CK(cudaGraphInstantiate(&ex, g, 0));
  CK(cudaGraphUpload(ex, st));

  const char* bgname[3] = {"idle", "d2h", "h2d"};
  const char* opname[5] = {"nothing", "timing_event", "notiming_event", "wait_done_event", "two_timing_events"};
  for (int bg = 0; bg < 3; bg++) {
    for (int op = 0; op < 5; op++) {
      std::vector<double> gaps;
      for (int rep = 0; rep < 6; rep++) {
        if (bg == 1) CK(cudaMemcpyAsync(hdst, dsrc, big, cudaMemcpyDeviceToHost, cp));
        if (bg == 2) CK(cudaMemcpyAsync(ddst, hsrc, big, cudaMemcpyHostToDevice, cp));
        stamp<<<1, 1, 0, st>>>(t + 0);  // warm-up kernel so the next pair starts on a busy link
        stamp<<<1, 1, 0, st>>>(t + 1);
        if (op == 1) CK(cudaEventRecord(et, st));
        if (op == 2) CK(cudaEventRecord(ent, st));
        if (op == 3) CK(cudaStreamWaitEvent(st, done, 0));
        if (op == 4) { CK(cudaEventRecord(et, st)); CK(cudaEventRecord(ga, st)); }
        stamp<<<1, 1, 0, st>>>(t + 2);
        CK(cudaStreamSynchronize(st));
        if (rep) gaps.push_back((t[2] - t[1]) / 1000.0);
        CK(cudaStreamSynchronize(cp));
      }
      std::sort(gaps.begin(), gaps.end());
      printf("{\"bg\": \"%s\", \"between_two_kernels\": \"%s\", \"gap_us_median\": %.2f, \"min\": %.2f, \"max\": %.2f}\n",
             bgname[bg], opname[op], gaps[gaps.size() / 2], gaps.front(), gaps.back());
    }
    // graph with event-record nodes between stamp kernels
    std::vector<double> g1, g2, ev;
    for (int rep = 0; rep < 6; rep++) {
      if (bg == 1) CK(cudaMemcpyAsync(hdst, dsrc, big, cudaMemcpyDeviceToHost, cp));
      if (bg == 2) CK(cudaMemcpyAsync(ddst, hsrc, big, cudaMemcpyHostToDevice, cp));
      stamp<<<1, 1, 0, st>>>(t + 0);
      CK(cudaGraphLaunch(ex, st));
      CK(cudaStreamSynchronize(st));
      uint64_t h[3];
      CK(cudaMemcpy(h, td, 24, cudaMemcpyDeviceToHost));
      float e = 0;
      CK(cudaEventElapsedTime(&e, ga, gb));
      if (rep) {
        g1.push_back((h[1] - h[0]) / 1000.0);
        g2.push_back((h[2] - h[1]) / 1000.0);
        ev.push_back(e * 1000.0);
      }
      CK(cudaStreamSynchronize(cp));
    }
    std::sort(g1.begin(), g1.end());
    std::sort(g2.begin(), g2.end());
    std::sort(ev.begin(), ev.end());
    printf("{\"bg\": \"%s\", \"graph\": \"stamp->evnode->stamp->evnode->stamp\", \"k0_to_k1_us\": %.2f, "
           "\"k1_to_k2_us\": %.2f, \"evnode_elapsed_us\": %.2f, \"evnode_elapsed_min\": %.2f, \"evnode_elapsed_max\": %.2f}\n",
           bgname[bg], g1[g1.size() / 2], g2[g2.size() / 2], ev[ev.size() / 2], ev.front(), ev.back());
  }
  // (a) the same stamp pairs writing DEVICE memory: is a kernel boundary during a copy expensive
  //     in itself, or only after a kernel that wrote host memory?
  // (b) timing events recorded on a side stream that waits for non-timing markers recorded on the
  //     launching stream around a 50 us kernel: accurate, and does the launching stream stall?
  cudaStream_t side;
  CK(cudaStreamCreateWithFlags(&side, cudaStreamNonBlocking));
  cudaEvent_t m0, m1, s0, s1;
  CK(cudaEventCreateWithFlags(&m0, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&m1, cudaEventDisableTiming));
  CK(cudaEventCreate(&s0));
  CK(cudaEventCreate(&s1));
  for (int bg = 0; bg < 3; bg++) {
    std::vector<double> gd, kern, side_ev, main_gap;
    for (int rep = 0; rep < 7; rep++) {
      if (bg == 1) CK(cudaMemcpyAsync(hdst, dsrc, big, cudaMemcpyDeviceToHost, cp));
      if (bg == 2) CK(cudaMemcpyAsync(ddst, hsrc, big, cudaMemcpyHostToDevice, cp));
      stamp<<<1, 1, 0, st>>>(td + 0);
      stamp<<<1, 1, 0, st>>>(td + 1);
      stamp<<<1, 1, 0, st>>>(td + 2);
      CK(cudaEventRecord(m0, st));
      CK(cudaStreamWaitEvent(side, m0, 0));
      CK(cudaEventRecord(s0, side));
      spin<<<1, 1, 0, st>>>(50000, td + 4);
      CK(cudaEventRecord(m1, st));
      CK(cudaStreamWaitEvent(side, m1, 0));
      CK(cudaEventRecord(s1, side));
      stamp<<<1, 1, 0, st>>>(td + 3);
      CK(cudaStreamSynchronize(st));
      CK(cudaStreamSynchronize(side));
      uint64_t h[6];
      CK(cudaMemcpy(h, td, 48, cudaMemcpyDeviceToHost));
      float e = 0;
      CK(cudaEventElapsedTime(&e, s0, s1));
      if (rep) {
        gd.push_back((h[2] - h[1]) / 1000.0);
        kern.push_back((h[5] - h[4]) / 1000.0);
        side_ev.push_back(e * 1000.0);
        main_gap.push_back((h[3] - h[2]) / 1000.0);
      }
      CK(cudaStreamSynchronize(cp));
    }
    for (auto* v : {&gd, &kern, &side_ev, &main_gap}) std::sort(v->begin(), v->end());
    printf("{\"bg\": \"%s\", \"device_stamp_boundary_us\": %.2f, \"spin_kernel_us\": %.2f, "
           "\"side_stream_events_us\": %.2f, \"side_min\": %.2f, \"side_max\": %.2f, "
           "\"main_stream_stamp_to_stamp_around_spin_us\": %.2f}\n",
           bgname[bg], gd[gd.size() / 2], kern[kern.size() / 2], side_ev[side_ev.size() / 2], side_ev.front(),
           side_ev.back(), main_gap[main_gap.size() / 2]);
  }
  printf("OK\n");
  return 0;
}
