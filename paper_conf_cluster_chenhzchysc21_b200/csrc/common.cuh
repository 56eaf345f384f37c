// common.cuh — shared device helpers for the CSWAP sm_100a kernels.
//
// Container v1 geometry, the epoch-tagged per-tile status words polled by the
// persistent ZVC compress, TMA bulk-copy / mbarrier wrappers and small PTX memory-order helpers.
#pragma once
#include <cstdlib>
#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

namespace cswap {

constexpr int kThreads = 256;          // every tile kernel: 8 warps
constexpr int kWarps = kThreads / 32;
constexpr uint32_t kTileBytes = 32768; // one tile = 32 KiB of raw input (8192 f32 / 16384 f16)
constexpr uint32_t kEpochs = 1u << 14; // status epoch tag width (14 bits)

enum : int { kNone = 0, kZVC = 1, kRLE = 2, kCSR = 3, kLZ4 = 4 };
enum : uint32_t { kErrOK = 0, kErrCorrupt = 5 };

__host__ __device__ __forceinline__ uint64_t a16(uint64_t x) { return (x + 15) & ~uint64_t(15); }
__host__ __device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__host__ __device__ __forceinline__ uint32_t umin32(uint32_t a, uint32_t b) { return a < b ? a : b; }
__host__ __device__ __forceinline__ uint64_t umax64(uint64_t a, uint64_t b) { return a > b ? a : b; }
__host__ __device__ __forceinline__ uint64_t cdiv(uint64_t a, uint64_t b) { return (a + b - 1) / b; }
__host__ __device__ __forceinline__ uint64_t data_start(uint32_t K) { return a16(64 + 8ull * K); }
__host__ __device__ __forceinline__ uint64_t frame_len(uint64_t n, uint64_t F, uint64_t k) {
  uint64_t s = k * F;
  return (n - s) < F ? (n - s) : F;
}

// ---- scratch shared by one launch sequence (leased per operation by api.cu) ----
struct Scratch {
  uint64_t* status;       // per-tile status word: value<<16 | epoch<<2 | flag
  uint32_t* tickets;      // per-epoch tile-ticket counters (zeroed slots)
  uint64_t* aux;          // per-frame / per-block u64 scratch (frame starts, block offsets ...)
  uint64_t* aux2;         // second per-frame / per-tile array
  uint32_t* err;          // device error word (first error wins)
  uint64_t* tbuf;         // per-tile u64 array for multi-kernel codecs (never epoch-tagged)
  uint64_t* tbuf2;        // second per-tile array, 32 bytes per tile (u64, or CSR: u32[8] slab counts)
  uint64_t* aux3;         // third per-frame u64 array (run / non-zero totals)
  uint64_t* zacc;         // persistent ZVC compress accumulators (zero between launches; cap_aux)
  uint64_t cap_tiles, cap_aux;
  // swap-out progress (NULL outside cswap_swap_out): u64[K], host-mapped pinned memory when
  // frames are published one by one from inside the kernel, else device memory that the library
  // copies to the host words after the group; the compress group stores kProgReady | (end offset
  // of frame k in the container) once every byte of frame k (and its frame-table entry) is in
  // device memory, so the host can start that frame's D2H
  uint64_t* prog;
  // ZVC compress only: 1 = publish each frame as soon as it is complete (the producer warps),
  // 2 = the last CTA publishes every frame once the kernel is done (no extra launch)
  uint32_t prog_mode;
  // kernel timing (NULL unless cswap_set_kernel_timing): device u64[2] = {CTA 0's start, the
  // last CTA's finish} in %globaltimer ns, written by the persistent ZVC compress
  uint64_t* kclock;
};

// programmatic dependent launch: wait until the preceding kernel in the stream has completed and
// its memory is visible (a no-op when the kernel was launched without the PDL attribute)
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
// let the next kernel of the stream (launched with the PDL attribute) start now: its CTAs become
// resident and block in pdl_wait() until this grid has completed
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
constexpr uint64_t kProgReady = 1ull << 63;

// Publish "frame k complete, ends at byte `end`" to host-mapped memory.  The caller has made the
// frame's stores visible at gpu scope (acq_rel chain or a kernel boundary); the copy engine
// that the host then starts reads device memory through L2, so no system-scope fence is needed
// (a fence.sys would wait behind the PCIe write queue of the D2H copies already in flight).
__device__ __forceinline__ void publish_frame(uint64_t* prog, uint32_t k, uint64_t end) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(prog + k), "l"(end | kProgReady) : "memory");
}

// ---- memory-order helpers -------------------------------------------------------------
__device__ __forceinline__ uint64_t ld_acquire(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(uint64_t* p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// Polling load: relaxed at gpu scope (no L1 invalidation, unlike ld.acquire which emits
// CCTL.IVALL).  Status words carry their payload, so relaxed reads are sufficient for them.
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

constexpr uint64_t kFlagA = 1, kFlagP = 2;
__device__ __forceinline__ uint64_t make_status(uint64_t value, uint32_t epoch, uint64_t flag) {
  return (value << 16) | (uint64_t(epoch) << 2) | flag;
}
__device__ __forceinline__ uint32_t status_flag(uint64_t s, uint32_t epoch) {
  return (uint32_t(s >> 2) & (kEpochs - 1)) == epoch ? uint32_t(s & 3) : 0u;
}
__device__ __forceinline__ uint64_t status_value(uint64_t s) { return s >> 16; }

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__device__ __forceinline__ void set_error(uint32_t* err, uint32_t code) {
  if (err) atomicCAS(err, 0u, code);
}

// ---- bulk async copy (TMA 1-D: cp.async.bulk global -> shared, mbarrier completion) -----
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(bar));
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(bar));
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  uint32_t d = static_cast<uint32_t>(__cvta_generic_to_shared(smem_dst));
  uint32_t b = static_cast<uint32_t>(__cvta_generic_to_shared(bar));
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d),
      "l"(gsrc), "r"(bytes), "r"(b)
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(bar));
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, 1000000;\n"  // suspend up to 1 ms per try
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(a),
      "r"(phase)
      : "memory");
}

// Wait with exponential __nanosleep backoff (32 ns .. max_ns) between non-blocking phase tests:
// for warps whose wait is off the critical path (a polling warp issues an instruction every ~20
// cycles even with try_wait's suspend hint, taking issue slots from the warps that do the work)
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t phase) {
  uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(bar)), ok;
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      "selp.u32 %0, 1, 0, p;\n"
      "}\n"
      : "=r"(ok)
      : "r"(a), "r"(phase)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t phase, uint32_t max_ns) {
  uint32_t ns = 32;
  while (!mbar_test(bar, phase)) {
    __nanosleep(ns);
    ns = ns < max_ns ? ns * 2 : max_ns;
  }
}

// ---- vector helpers -------------------------------------------------------------------
__device__ __forceinline__ uint4 ldg_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
// shared-memory loads by 32-bit shared-window address (no generic->shared conversion per load)
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint4 lds_v4(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ void stg_stream(uint4* p, uint4 v) {
  asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}

// Copy a slab's compacted non-zeros (cnt words of W bytes at shared sv) to dst: element stores up
// to the destination's next 16-byte boundary, then 16-byte stores whose source is the smem slab
// funnel-shifted by that head (k whole words + r bits, warp-uniform, so one of four unrolled
// bodies runs), then the element tail.  Called by `stride` threads (a warp: stride 32, idx =
// lane; a block: stride blockDim.x, idx = threadIdx.x); sv is 16-byte aligned with >= 16
// readable bytes past the last word.
template <typename T>
__device__ __forceinline__ void emit_words(const T* sv, uint32_t cnt, uint8_t* dst, uint32_t idx, uint32_t stride) {
  T* d = reinterpret_cast<T*>(dst);
  const uint32_t nbytes = cnt * sizeof(T);
  const uint32_t h = umin32((16u - (uint32_t(reinterpret_cast<uintptr_t>(dst)) & 15u)) & 15u, nbytes);
  const uint32_t nb = (nbytes - h) >> 4, tail = h + 16 * nb;
  if (idx < h / sizeof(T)) d[idx] = sv[idx];
  if (idx < (nbytes - tail) / sizeof(T)) d[tail / sizeof(T) + idx] = sv[tail / sizeof(T) + idx];
  const uint32_t sa = uint32_t(__cvta_generic_to_shared(sv));
  uint4* dv = reinterpret_cast<uint4*>(dst + h);
  auto body = [&](auto kk) {
    constexpr int k = decltype(kk)::value;
    const uint32_t r = (h & 3u) * 8u;
#pragma unroll 2
    for (uint32_t q = idx; q < nb; q += stride) {
      const uint4 A = lds_v4(sa + 16 * q), B = lds_v4(sa + 16 * q + 16);
      const uint32_t w[8] = {A.x, A.y, A.z, A.w, B.x, B.y, B.z, B.w};
      stg_stream(dv + q, make_uint4(__funnelshift_r(w[k], w[k + 1], r), __funnelshift_r(w[k + 1], w[k + 2], r),
                                    __funnelshift_r(w[k + 2], w[k + 3], r), __funnelshift_r(w[k + 3], w[k + 4], r)));
    }
  };
  switch (h >> 2) {
    case 0: body(std::integral_constant<int, 0>{}); break;
    case 1: body(std::integral_constant<int, 1>{}); break;
    case 2: body(std::integral_constant<int, 2>{}); break;
    default: body(std::integral_constant<int, 3>{}); break;
  }
}

// Write the 64-byte container header (one thread).
__device__ __forceinline__ void write_header(uint8_t* out, int codec, int dtype, uint64_t n, uint64_t F,
                                             uint32_t K, uint32_t param, uint64_t total) {
  uint32_t* o32 = reinterpret_cast<uint32_t*>(out);
  uint64_t* o64 = reinterpret_cast<uint64_t*>(out);
  o32[0] = 0x50575343u;                                             // "CSWP"
  o32[1] = 1u | (uint32_t(codec) << 16) | (uint32_t(dtype) << 24);  // version 1, codec, dtype
  o64[1] = n;
  o64[2] = F;
  o32[6] = K;
  o32[7] = param;
  o64[4] = total;
  o64[5] = 0;
  o64[6] = 0;
  o64[7] = 0;
}

// Programmatic dependent launch (PDL) for the kernels of a launch group: CSWAP_PDL=0 launches plainly (A/B).
// Every kernel launched this way calls pdl_wait() before reading its predecessor's output.
inline bool pdl_enabled() {
  static int p = -1;
  if (p < 0) {
    const char* e = getenv("CSWAP_PDL");
    p = (e && e[0] == '0') ? 0 : 1;
  }
  return p == 1;
}
template <typename... KArgs, typename... Args>
inline cudaError_t pdl_launch(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                              Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}
#define CUDA_TRY_LAUNCH(x)                    \
  do {                                        \
    const cudaError_t e_ = (x);               \
    if (e_ != cudaSuccess) return e_;         \
  } while (0)


}  // namespace cswap
