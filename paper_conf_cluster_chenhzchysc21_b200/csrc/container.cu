// container.cu — codec-independent kernels: container header/prep, NONE frames, sparsity probe.
//
// Container v1 layout: DESIGN.md §3.  Probe: PAPER.md:118 (§IV-A, the tensor profiler collects
// sparsity), :327 (§V-E, "CSWAP utilizes GPU multi-cores to profile tensor sparsity"); window
// design DESIGN.md R15 / §3.3.
#include "common.cuh"
#include "kernels.h"

namespace cswap {

// ---- header-only container (n = 0) and NONE header ------------------------------------------
__global__ void header_kernel(uint8_t* out, int codec, int dtype, uint64_t n, uint64_t F, uint32_t param,
                              uint64_t* out_size) {
  const uint32_t K = uint32_t(cdiv(n, F));
  const int w = dtype == 0 ? 4 : 2;
  uint64_t total = data_start(K);
  for (uint32_t k = threadIdx.x; k < K; k += blockDim.x) {
    const uint64_t fb = a16(uint64_t(w) * frame_len(n, F, k));
    reinterpret_cast<uint64_t*>(out + 64)[k] = fb;
  }
  if (threadIdx.x == 0) {
    for (uint32_t k = 0; k < K; k++) total += a16(uint64_t(w) * frame_len(n, F, k));
    write_header(out, codec, dtype, n, F, K, param, total);
    for (uint64_t b = 64 + 8ull * K; b < data_start(K); b += 8) *reinterpret_cast<uint64_t*>(out + b) = 0;
    if (K) {  // zero the pad after the last raw frame
      const uint64_t end = data_start(K) + uint64_t(w) * n;
      for (uint64_t b = end; b < total; b++) out[b] = 0;
    }
    *out_size = total;
  }
}

cudaError_t launch_header_only(uint8_t* out, int codec, int dtype, uint64_t F, uint32_t param, uint64_t* out_size,
                               cudaStream_t st) {
  header_kernel<<<1, 32, 0, st>>>(out, codec, dtype, 0, F, param, out_size);
  return cudaGetLastError();
}

cudaError_t launch_none_compress(const void* in, uint64_t n, int w, uint64_t F, int dtype, uint8_t* out,
                                 uint64_t* out_size, cudaStream_t st) {
  const uint32_t K = uint32_t(cdiv(n, F));
  // non-last frames are F*w bytes (a multiple of 16), so the raw frames are one contiguous run
  cudaError_t e = cudaMemcpyAsync(out + data_start(K), in, n * w, cudaMemcpyDeviceToDevice, st);
  if (e != cudaSuccess) return e;
  header_kernel<<<1, 256, 0, st>>>(out, kNone, dtype, n, F, 0, out_size);
  return cudaGetLastError();
}

// ---- frame table finalize (multi-pass codecs): frame_bytes[k] in fbytes[k] -> frame table,
// frame starts (fstart[k]), header, padding, *out_size.  One CTA.
__global__ void __launch_bounds__(1024) finalize_kernel(uint8_t* out, int codec, int dtype, uint64_t n, uint64_t F,
                                                        uint32_t param, const uint64_t* fbytes, uint64_t* fstart,
                                                        uint64_t* out_size) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  __shared__ uint64_t s_w[33];
  const uint32_t K = uint32_t(cdiv(n, F));
  const uint64_t base = data_start(K);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t carry = 0;
  for (uint32_t c = 0; c < K; c += blockDim.x) {
    const uint32_t k = c + threadIdx.x;
    const uint64_t fb = k < K ? fbytes[k] : 0;
    uint64_t inc = fb;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
    if (lane == 31) s_w[warp] = inc;
    __syncthreads();
    if (threadIdx.x == 0) {
      uint64_t acc = 0;
      for (int w = 0; w < int(blockDim.x / 32); w++) {
        const uint64_t x = s_w[w];
        s_w[w] = acc;
        acc += x;
      }
      s_w[32] = acc;
    }
    __syncthreads();
    if (k < K) {
      fstart[k] = base + carry + s_w[warp] + inc - fb;
      reinterpret_cast<uint64_t*>(out + 64)[k] = fb;
    }
    carry += s_w[32];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    const uint64_t total = base + carry;
    write_header(out, codec, dtype, n, F, K, param, total);
    for (uint64_t b = 64 + 8ull * K; b < base; b += 8) *reinterpret_cast<uint64_t*>(out + b) = 0;
    *out_size = total;
  }
}

cudaError_t launch_finalize(uint8_t* out, int codec, int dtype, uint64_t n, uint64_t F, uint32_t param,
                            const Scratch& sc, uint64_t* out_size, cudaStream_t st) {
  CUDA_TRY_LAUNCH(pdl_launch(finalize_kernel, dim3(1), dim3(1024), 0, st, out, codec, dtype, n, F, param, sc.aux2, sc.aux, out_size));
  return cudaGetLastError();
}

// ---- zero fill of small scratch arrays (kept off the copy engines: a cudaMemsetAsync may be
// queued behind a long D2H/H2D on the same engine) --------------------------------------------
__global__ void zero_words_kernel(uint32_t* p, uint64_t words) {
  for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < words; i += uint64_t(gridDim.x) * blockDim.x)
    p[i] = 0u;
}

cudaError_t launch_zero_words(void* p, uint64_t words, cudaStream_t st) {
  if (!words) return cudaSuccess;
  const uint64_t blocks = std::min<uint64_t>((words + 255) / 256, 1184);
  zero_words_kernel<<<unsigned(blocks), 256, 0, st>>>(static_cast<uint32_t*>(p), words);
  return cudaGetLastError();
}

// ---- error word merge (device scratch word -> caller's word, first error wins) ---------------
__global__ void err_merge_kernel(const uint32_t* src, uint32_t* dst) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  const uint32_t v = *src;
  if (v) atomicCAS(dst, 0u, v);
}

cudaError_t launch_err_merge(const uint32_t* src, uint32_t* dst, cudaStream_t st) {
  CUDA_TRY_LAUNCH(pdl_launch(err_merge_kernel, dim3(1), dim3(1), 0, st, src, dst));
  return cudaGetLastError();
}

// ---- prep: validate the header and scan the frame table --------------------------------------
__device__ __forceinline__ uint64_t block_excl_scan_u64(uint64_t v, uint64_t* s_warp, uint64_t* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  uint64_t inc = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) s_warp[warp] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t acc = 0;
    for (int w = 0; w < nw; w++) {
      uint64_t x = s_warp[w];
      s_warp[w] = acc;
      acc += x;
    }
    s_warp[nw] = acc;
  }
  __syncthreads();
  const uint64_t r = s_warp[warp] + inc - v;
  *total = s_warp[nw];
  __syncthreads();
  return r;
}

__global__ void __launch_bounds__(1024) prep_kernel(const uint8_t* in, uint64_t in_size, int codec, int dtype,
                                                    uint64_t n, uint64_t F, uint32_t param, uint64_t* fstart,
                                                    uint64_t* fbytes, uint32_t* err, int reset_err) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  __shared__ int s_ok;
  __shared__ uint64_t s_total;
  __shared__ uint64_t s_warp[33];
  const uint32_t K = uint32_t(cdiv(n, F));
  if (threadIdx.x == 0) {
    if (reset_err) *err = 0;  // first kernel of the decode: clears the lease's error word
    int ok = in_size >= 64;
    if (ok) {
      const uint32_t* h32 = reinterpret_cast<const uint32_t*>(in);
      const uint64_t* h64 = reinterpret_cast<const uint64_t*>(in);
      ok = h32[0] == 0x50575343u && (h32[1] & 0xFFFFu) == 1u && int((h32[1] >> 16) & 0xFF) == codec &&
           int(h32[1] >> 24) == dtype && h64[1] == n && h64[2] == F && h32[6] == K && h32[7] == param;
      s_total = h64[4];
      ok = ok && s_total <= in_size && s_total >= data_start(K);
    }
    s_ok = ok;
    if (!ok) set_error(err, kErrCorrupt);
  }
  __syncthreads();
  if (!s_ok) {
    for (uint32_t k = threadIdx.x; k < K; k += blockDim.x) fstart[k] = fbytes[k] = 0;
    return;
  }
  const uint64_t* table = reinterpret_cast<const uint64_t*>(in + 64);
  const uint64_t base = data_start(K);
  uint64_t carry = 0;
  bool bad = false;
  for (uint32_t c = 0; c < K; c += blockDim.x) {
    const uint32_t k = c + threadIdx.x;
    const uint64_t fb = k < K ? table[k] : 0;
    bad |= (fb & 15) != 0 || fb > s_total;
    uint64_t tot;
    const uint64_t ex = block_excl_scan_u64(fb, s_warp, &tot);
    if (k < K) {
      fstart[k] = base + carry + ex;
      fbytes[k] = fb;
    }
    carry += tot;
  }
  // a bad frame table leaves every frame empty (start 0, 0 bytes): single-pass decoders, which
  // cannot stop early without stalling their successors, then see a size mismatch and read nothing
  __shared__ int s_bad;
  if (threadIdx.x == 0) s_bad = 0;
  __syncthreads();
  if (bad || (threadIdx.x == 0 && base + carry != s_total)) s_bad = 1;
  __syncthreads();
  if (s_bad) {
    if (threadIdx.x == 0) set_error(err, kErrCorrupt);
    for (uint32_t k = threadIdx.x; k < K; k += blockDim.x) fstart[k] = fbytes[k] = 0;
  }
}

cudaError_t launch_prep(const uint8_t* in, uint64_t in_size, int codec, int dtype, uint64_t n, uint64_t F,
                        uint32_t param, const Scratch& sc, uint32_t* err, bool reset_err, cudaStream_t st) {
  timing_kernel_start(st);
  CUDA_TRY_LAUNCH(pdl_launch(prep_kernel, dim3(1), dim3(1024), 0, st, in, in_size, codec, dtype, n, F, param, sc.aux, sc.aux2, err, reset_err ? 1 : 0));
  return cudaGetLastError();
}

// ---- timing stamps: one thread writes %globaltimer (ns) into a device slot; the group's first
// stamp also clears the slot's end stamp and container-size word (slots are reused)
__global__ void stamp_kernel(unsigned long long* dst, int first) {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  dst[0] = t;
  if (first) {  // slot: [0] start, [1] end, [2] container size, [3..4] kernel clock (Scratch::kclock)
    dst[1] = dst[2] = dst[4] = 0;
    dst[3] = ~0ull;
  }
}

cudaError_t launch_stamp(uint64_t* dst, cudaStream_t st, bool first) {
  stamp_kernel<<<1, 1, 0, st>>>(reinterpret_cast<unsigned long long*>(dst), first ? 1 : 0);
  return cudaGetLastError();
}

// ---- NONE decompress: frames are raw; check sizes, copy -----------------------------------
__global__ void none_check_kernel(uint64_t n, uint64_t F, int w, const uint64_t* fbytes, uint32_t* err) {
  const uint32_t K = uint32_t(cdiv(n, F));
  for (uint32_t k = threadIdx.x; k < K; k += blockDim.x)
    if (fbytes[k] != a16(uint64_t(w) * frame_len(n, F, k))) set_error(err, kErrCorrupt);
}

cudaError_t launch_none_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, const Scratch& sc,
                                   uint32_t* err, cudaStream_t st) {
  const uint32_t K = uint32_t(cdiv(n, F));
  none_check_kernel<<<1, 256, 0, st>>>(n, F, w, sc.aux2, err);
  return cudaMemcpyAsync(out, in + data_start(K), n * w, cudaMemcpyDeviceToDevice, st);
}

// ---- sparsity probe ----------------------------------------------------------------------
constexpr int kProbeW = 256, kProbeSw = 1024;

template <typename T>
__global__ void __launch_bounds__(kThreads) probe_kernel(const T* __restrict__ x, uint64_t n, uint32_t pieces,
                                                         bool single, uint64_t* partial, uint32_t* done,
                                                         uint64_t* counts3, uint32_t tag) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t z = 0, zr = 0, bd = 0;
  for (uint32_t p = blockIdx.x * kWarps + warp; p < pieces; p += gridDim.x * kWarps) {
    uint64_t start, ws;
    if (single) { start = uint64_t(p) * kProbeW; ws = 0; }
    else { start = uint64_t(p) * (n - kProbeW) / (kProbeSw - 1); ws = start; }
    const uint64_t end = single ? umin64(start + kProbeW, n) : start + kProbeW;
    uint32_t v[8];
    const uint64_t i0 = start + lane * 8;
#pragma unroll
    for (int i = 0; i < 8; i++) v[i] = (i0 + i < end) ? uint32_t(x[i0 + i]) : 0u;
    uint32_t prev = __shfl_up_sync(0xffffffffu, v[7], 1);
    if (lane == 0) prev = start > ws ? uint32_t(x[start - 1]) : 0u;
#pragma unroll
    for (int i = 0; i < 8; i++) {
      const uint64_t gi = i0 + i;
      if (gi < end) {
        const bool first = gi == ws;
        z += v[i] == 0;
        zr += v[i] == 0 && (first || prev != 0);
        bd += !first && v[i] != prev;
      }
      prev = v[i];
    }
  }
  z = warp_sum_u64(z);
  zr = warp_sum_u64(zr);
  bd = warp_sum_u64(bd);
  __shared__ uint64_t s[kWarps][3];
  __shared__ bool s_last;
  if (lane == 0) { s[warp][0] = z; s[warp][1] = zr; s[warp][2] = bd; }
  __syncthreads();
  if (threadIdx.x < 3) {
    uint64_t a = 0;
    for (int w = 0; w < kWarps; w++) a += s[w][threadIdx.x];
    partial[blockIdx.x * 3 + threadIdx.x] = a;
  }
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) s_last = atomicAdd(done, 1u) == gridDim.x - 1;
  __syncthreads();
  if (s_last && warp < 3) {  // warp c sums counter c over the CTAs' partials
    __threadfence();
    uint64_t a = 0;
    for (uint32_t b = lane; b < gridDim.x; b += 32) a += __ldcg(partial + b * 3 + warp);
    a = warp_sum_u64(a);
    // one 64-bit store per count, tagged with this launch's 16-bit tag: the host polls the three
    // words in mapped memory until all carry the tag (no completion event to wait for)
    if (lane == 0) counts3[warp] = (a << 16) | tag;
  }
}

cudaError_t launch_probe(const void* in, uint64_t n, int w, uint64_t* counts3, uint32_t tag, const Scratch& sc,
                         uint32_t epoch, cudaStream_t st) {
  const bool single = n <= uint64_t(kProbeW) * kProbeSw;
  const uint32_t pieces = single ? uint32_t(cdiv(n, kProbeW)) : kProbeSw;
  const uint32_t grid = uint32_t(umin64(cdiv(pieces, kWarps), 128));
  timing_kernel_start(st);
  if (w == 4)
    probe_kernel<uint32_t><<<grid, kThreads, 0, st>>>(static_cast<const uint32_t*>(in), n, pieces, single, sc.aux2,
                                                      sc.tickets + epoch, counts3, tag);
  else
    probe_kernel<uint16_t><<<grid, kThreads, 0, st>>>(static_cast<const uint16_t*>(in), n, pieces, single, sc.aux2,
                                                      sc.tickets + epoch, counts3, tag);
  return cudaGetLastError();
}

}  // namespace cswap

namespace cswap {
// Swap-out progress for the multi-pass codecs (RLE, CSR, LZ4, NONE): launched after the group's
// last kernel, so every frame is complete; writes kProgReady | end offset of each frame from the
// container's frame table (one CTA: per-thread chunk sums, block scan, per-thread writes).
__global__ void __launch_bounds__(1024) publish_frames_kernel(const uint8_t* out, uint32_t K, uint64_t* prog) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  __shared__ uint64_t s_w[33];
  const uint64_t* fb = reinterpret_cast<const uint64_t*>(out + 64);
  const uint32_t per = (K + blockDim.x - 1) / blockDim.x, k0 = threadIdx.x * per, k1 = umin32(K, k0 + per);
  uint64_t sum = 0;
  for (uint32_t k = k0; k < k1; k++) sum += fb[k];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t inc = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) s_w[warp] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t acc = 0;
    for (int w = 0; w < int(blockDim.x / 32); w++) {
      const uint64_t x = s_w[w];
      s_w[w] = acc;
      acc += x;
    }
  }
  __syncthreads();
  uint64_t end = data_start(K) + s_w[warp] + inc - sum;
  for (uint32_t k = k0; k < k1; k++) {
    end += fb[k];
    publish_frame(prog, k, end);
  }
}

cudaError_t launch_publish_frames(const uint8_t* out, uint32_t K, uint64_t* prog, cudaStream_t st) {
  if (!K) return cudaSuccess;
  CUDA_TRY_LAUNCH(pdl_launch(publish_frames_kernel, dim3(1), dim3(1024), 0, st, out, K, prog));
  return cudaGetLastError();
}
}  // namespace cswap
