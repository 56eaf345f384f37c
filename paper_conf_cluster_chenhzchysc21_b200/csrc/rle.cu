// rle.cu — run-length encoding for sm_100a.
//
// PAPER.md:220 (§IV-E): "RLE stores data sequences where the same value occurs in many
// consecutive positions as a single value and count".  Reading R4: a
// (length, value) pair for EVERY maximal run of bitwise-equal words; runs never cross frames.
// Frame payload: {u32 r, 12 zero bytes} | u32 lengths[r] pad16 | values[r] pad16.
//
// The values section starts after all r lengths, so a tile can only place its runs once the
// whole frame is counted; compress is therefore: count (run starts per tile + first start) ->
// per-frame scan (run offsets, next run start after each tile, r_k) -> frame table -> emit.
// Decompress: per-frame scan of the lengths into run start positions, then one CTA per output
// tile where every element finds its run by binary search.
#include "kernels.h"
#include "tile_common.cuh"

namespace cswap {

// run-start flag of tile element e: frame start, or differs from its predecessor
template <typename T>
__device__ __forceinline__ bool run_start(const T* s_x, uint32_t e, const TilePos& p, T prev) {
  if (e == 0) return p.j == 0 || s_x[0] != prev;
  return s_x[e] != s_x[e - 1];
}

template <typename T>
__global__ void __launch_bounds__(kThreads) rle_count_kernel(const T* __restrict__ in, uint64_t n, uint64_t F,
                                                             uint32_t tpf, Scratch sc) {
  using G = TileGeom<T>;
  __shared__ __align__(16) T s_x[G::TILE];
  __shared__ uint64_t s_tmp[33];
  const uint32_t t = blockIdx.x;
  const TilePos p = tile_pos<T>(t, n, F, tpf);
  const T* src = in + uint64_t(p.k) * F + p.tin;
  stage_tile<T>(s_x, src, p.te);
  const T prev = p.j ? src[-1] : T(0);
  uint32_t c = 0;
  uint64_t first = ~uint64_t(0);
  for (uint32_t e = threadIdx.x; e < p.te; e += blockDim.x) {
    if (run_start<T>(s_x, e, p, prev)) {
      c++;
      first = umin64(first, p.tin + e);
    }
  }
  c = block_sum_u32(c, reinterpret_cast<uint32_t*>(s_tmp));
  first = block_min_u64(first, s_tmp);
  if (threadIdx.x == 0) {
    sc.tbuf[t] = c;
    sc.tbuf2[t] = first;
  }
}

// one CTA per frame: run offsets per tile (tbuf), next run start after each tile (tbuf2),
// r_k (aux3), frame_bytes (aux2)
template <typename T>
__global__ void __launch_bounds__(1024) rle_scan_kernel(uint64_t n, uint64_t F, uint32_t tpf, Scratch sc) {
  using G = TileGeom<T>;
  __shared__ uint64_t s_tmp[33];
  const uint32_t k = blockIdx.x;
  const uint64_t Fk = frame_len(n, F, k);
  const uint32_t nt = uint32_t(cdiv(Fk, G::TILE));
  uint64_t* cnt = sc.tbuf + uint64_t(k) * tpf;
  uint64_t* nxt = sc.tbuf2 + uint64_t(k) * tpf;
  uint64_t carry = 0;
  for (uint32_t c0 = 0; c0 < nt; c0 += blockDim.x) {
    const uint32_t j = c0 + threadIdx.x;
    const uint64_t v = j < nt ? cnt[j] : 0;
    uint64_t tot;
    const uint64_t ex = block_excl_sum_u64(v, s_tmp, &tot);
    if (j < nt) cnt[j] = carry + ex;
    carry += tot;
  }
  // next run start after tile j = min(first start of tiles > j), else the frame end
  uint64_t after = Fk;
  for (int64_t c1 = int64_t(nt); c1 > 0; c1 -= blockDim.x) {
    const int64_t c0 = c1 - int64_t(blockDim.x) > 0 ? c1 - int64_t(blockDim.x) : 0;
    const int64_t j = c0 + threadIdx.x;
    const uint64_t v = j < c1 ? nxt[j] : ~uint64_t(0);
    uint64_t all;
    const uint64_t r = block_excl_suffix_min_u64(v, s_tmp, &all);
    if (j < c1) nxt[j] = umin64(r, after);
    after = umin64(after, all);
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    sc.aux3[k] = carry;
    sc.aux2[k] = 16 + a16(4 * carry) + a16(uint64_t(G::W) * carry);
  }
}

template <typename T>
__global__ void __launch_bounds__(kThreads) rle_emit_kernel(const T* __restrict__ in, uint64_t n, uint64_t F,
                                                            uint32_t tpf, uint8_t* __restrict__ out, Scratch sc) {
  using G = TileGeom<T>;
  __shared__ __align__(16) T s_x[G::TILE];
  __shared__ uint32_t s_wcnt[kWarps + 1];
  extern __shared__ __align__(16) uint16_t s_bpos[];  // run starts of the tile (tile-relative)
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t t = blockIdx.x;
  const TilePos p = tile_pos<T>(t, n, F, tpf);
  const T* src = in + uint64_t(p.k) * F + p.tin;
  stage_tile<T>(s_x, src, p.te);
  const T prev = p.j ? src[-1] : T(0);
  // warp w: elements [w*PER_WARP, (w+1)*PER_WARP) row by row; compact run starts warp-locally
  uint32_t cnt = 0;
  const uint32_t lt = (1u << lane) - 1u;
  uint16_t* wpos = s_bpos + warp * G::PER_WARP;
  for (int m = 0; m < G::ROWS; m++) {
    const uint32_t e = warp * G::PER_WARP + 32 * m + lane;
    const bool f = e < p.te && run_start<T>(s_x, e, p, prev);
    const uint32_t b = __ballot_sync(0xffffffffu, f);
    if (f) wpos[cnt + __popc(b & lt)] = uint16_t(e);
    cnt += __popc(b);
  }
  if (lane == 0) s_wcnt[warp] = cnt;
  __syncthreads();
  if (tid == 0) {
    uint32_t a = 0;
    for (int w = 0; w < kWarps; w++) {
      const uint32_t x = s_wcnt[w];
      s_wcnt[w] = a;
      a += x;
    }
    s_wcnt[kWarps] = a;
  }
  __syncthreads();
  const uint32_t total = s_wcnt[kWarps];
  const uint64_t run_off = sc.tbuf[t];
  const uint64_t next_start = sc.tbuf2[t];
  const uint64_t r_k = sc.aux3[p.k];
  const uint64_t fstart = sc.aux[p.k];
  uint32_t* lengths = reinterpret_cast<uint32_t*>(out + fstart + 16);
  uint8_t* values = out + fstart + 16 + a16(4 * r_k);
  // gather the warp lists into one ordered sequence: run q of the tile is in warp w's list at
  // q - s_wcnt[w]; write length and value of every run starting in this tile
  for (uint32_t q = tid; q < total; q += kThreads) {
    int w = 0;
    while (w + 1 < kWarps && s_wcnt[w + 1] <= q) w++;
    const uint32_t pos = s_bpos[w * G::PER_WARP + (q - s_wcnt[w])];
    uint64_t end;
    if (q + 1 < total) {
      int w2 = w;
      while (w2 + 1 < kWarps && s_wcnt[w2 + 1] <= q + 1) w2++;
      end = p.tin + s_bpos[w2 * G::PER_WARP + (q + 1 - s_wcnt[w2])];
    } else {
      end = next_start;
    }
    lengths[run_off + q] = uint32_t(end - (p.tin + pos));
    reinterpret_cast<T*>(values)[run_off + q] = s_x[pos];
  }
  if (tid == 0 && p.j == 0) {  // sub-header {u32 r, 12 zero bytes}
    uint32_t* h = reinterpret_cast<uint32_t*>(out + fstart);
    h[0] = uint32_t(r_k);
    h[1] = h[2] = h[3] = 0;
  }
  if (tid == kThreads - 1 && p.tin + p.te == p.Fk) {  // last tile of the frame: section pads
    for (uint64_t b = 16 + 4 * r_k; b < 16 + a16(4 * r_k); b += 4) *reinterpret_cast<uint32_t*>(out + fstart + b) = 0;
    const uint64_t vb = 16 + a16(4 * r_k);
    for (uint64_t b = vb + G::W * r_k; b < vb + a16(G::W * r_k); b += 2) *reinterpret_cast<uint16_t*>(out + fstart + b) = 0;
  }
}

uint32_t rle_tiles(uint64_t n, int w, uint64_t F) {
  const uint32_t TILE = kTileBytes / w;
  const uint32_t K = uint32_t(cdiv(n, F));
  const uint32_t tpf = uint32_t(cdiv(F, TILE));
  if (!K) return 0;
  return (K - 1) * tpf + uint32_t(cdiv(frame_len(n, F, K - 1), TILE));
}

template <typename T>
static cudaError_t rle_compress_t(const void* in, uint64_t n, uint64_t F, uint8_t* out, uint64_t* out_size,
                                  const Scratch& sc, int dtype, cudaStream_t st) {
  using G = TileGeom<T>;
  const uint32_t K = uint32_t(cdiv(n, F));
  const uint32_t tpf = uint32_t(cdiv(F, G::TILE));
  const uint32_t tiles = rle_tiles(n, sizeof(T), F);
  const T* x = static_cast<const T*>(in);
  timing_kernel_start(st);
  rle_count_kernel<T><<<tiles, kThreads, 0, st>>>(x, n, F, tpf, sc);
  rle_scan_kernel<T><<<K, 1024, 0, st>>>(n, F, tpf, sc);
  cudaError_t e = launch_finalize(out, kRLE, dtype, n, F, 0, sc, out_size, st);
  if (e != cudaSuccess) return e;
  const int smem = G::TILE * 2;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(rle_emit_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  rle_emit_kernel<T><<<tiles, kThreads, smem, st>>>(x, n, F, tpf, out, sc);
  return cudaGetLastError();
}

cudaError_t launch_rle_compress(const void* in, uint64_t n, int w, uint64_t F, uint8_t* out, uint64_t* out_size,
                                const Scratch& sc, uint32_t /*epoch*/, int dtype, cudaStream_t st) {
  return w == 4 ? rle_compress_t<uint32_t>(in, n, F, out, out_size, sc, dtype, st)
                : rle_compress_t<uint16_t>(in, n, F, out, out_size, sc, dtype, st);
}

// ------------------------------------------------------------------------------------------
// decompress
// ------------------------------------------------------------------------------------------
// one CTA per frame: validate, run start positions (frame-relative) into rs[k*F + i]
template <typename T>
__global__ void __launch_bounds__(1024) rle_dscan_kernel(const uint8_t* __restrict__ in, uint64_t n, uint64_t F,
                                                         uint32_t k0, uint32_t* rs, Scratch sc, uint32_t* err) {
  using G = TileGeom<T>;
  __shared__ uint64_t s_tmp[33];
  __shared__ int s_ok;
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const uint32_t k = k0 + blockIdx.x;
  const uint64_t Fk = frame_len(n, F, k);
  const uint64_t fstart = sc.aux[k], fb = sc.aux2[k];
  if (threadIdx.x == 0) {
    int ok = fb >= 16;
    uint64_t r = ok ? *reinterpret_cast<const uint32_t*>(in + fstart) : 0;
    ok = ok && r >= 1 && r <= Fk && fb == 16 + a16(4 * r) + a16(uint64_t(G::W) * r);
    sc.aux3[k] = ok ? r : 0;
    s_ok = ok;
    if (!ok) set_error(err, kErrCorrupt);
  }
  __syncthreads();
  if (!s_ok) return;
  const uint64_t r = sc.aux3[k];
  const uint32_t* len = reinterpret_cast<const uint32_t*>(in + fstart + 16);
  uint32_t* out = rs + uint64_t(k) * F;
  uint64_t carry = 0;
  bool bad = false;
  for (uint64_t c0 = 0; c0 < r; c0 += blockDim.x) {
    const uint64_t i = c0 + threadIdx.x;
    const uint64_t v = i < r ? len[i] : 0;
    bad |= i < r && v == 0;
    uint64_t tot;
    const uint64_t ex = block_excl_sum_u64(v, s_tmp, &tot);
    if (i < r) out[i] = uint32_t(umin64(carry + ex, Fk));
    carry += tot;
  }
  if (bad || carry != Fk) set_error(err, kErrCorrupt);
}

// one CTA per output tile: element e -> run = last start <= e (binary search), value of that run
template <typename T>
__global__ void __launch_bounds__(kThreads) rle_expand_kernel(const uint8_t* __restrict__ in, T* __restrict__ outp,
                                                              uint64_t n, uint64_t F, uint32_t tpf, uint32_t k0,
                                                              const uint32_t* rs, Scratch sc, uint32_t* err) {
  using G = TileGeom<T>;
  __shared__ uint64_t s_lo, s_hi;
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const uint32_t t = blockIdx.x + k0 * tpf;
  const TilePos p = tile_pos<T>(t, n, F, tpf);
  const uint64_t r = sc.aux3[p.k];
  if (r == 0) return;
  const uint32_t* st = rs + uint64_t(p.k) * F;
  const T* values = reinterpret_cast<const T*>(in + sc.aux[p.k] + 16 + a16(4 * r));
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  // warps 0/1: 32-ary search for the runs holding the tile's first / last element
  if (warp < 2) {
    const uint64_t target = warp == 0 ? p.tin : p.tin + p.te - 1;
    uint64_t lo = 0, hi = r;  // answer in [lo, hi): last i with st[i] <= target
    while (hi - lo > 1) {
      const uint64_t span = hi - lo;
      const uint64_t probe = lo + (span * uint64_t(lane)) / 32;
      const bool le = st[probe] <= target;
      const uint32_t m = __ballot_sync(0xffffffffu, le);
      const int last = 31 - __clz(m);  // lane 0 always satisfies (st[lo] <= target)
      const uint64_t nlo = lo + (span * uint64_t(last)) / 32;
      const uint64_t nhi = last == 31 ? hi : lo + (span * uint64_t(last + 1)) / 32;
      lo = nlo;
      hi = nhi > nlo ? nhi : nlo + 1;
    }
    if (lane == 0) {
      if (warp == 0) s_lo = lo;
      else s_hi = lo;
    }
  }
  __syncthreads();
  const uint64_t rlo = s_lo, rhi = s_hi;
  T* dst = outp + uint64_t(p.k) * F + p.tin;
  for (uint32_t e = threadIdx.x; e < p.te; e += blockDim.x) {
    const uint64_t pos = p.tin + e;
    uint64_t lo = rlo, hi = rhi + 1;
    while (hi - lo > 1) {
      const uint64_t mid = (lo + hi) / 2;
      if (st[mid] <= pos) lo = mid;
      else hi = mid;
    }
    dst[e] = values[lo];
  }
}

cudaError_t launch_rle_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t k0,
                                  uint32_t k1, const Scratch& sc, uint32_t /*epoch*/, uint32_t* err, cudaStream_t st) {
  if (k1 <= k0) return cudaSuccess;
  const uint32_t TILE = kTileBytes / w;
  const uint32_t tpf = uint32_t(cdiv(F, TILE));
  uint32_t* rs = nullptr;  // run starts, indexed k*F + i (i < r_k <= F_k): at most n entries
  cudaError_t e = cudaMallocAsync(&rs, n * 4 + 64, st);
  if (e != cudaSuccess) return e;
  const uint32_t tiles = (k1 - 1 - k0) * tpf + uint32_t(cdiv(frame_len(n, F, k1 - 1), TILE));
  if (w == 4) {
    timing_kernel_start(st);
    rle_dscan_kernel<uint32_t><<<k1 - k0, 1024, 0, st>>>(in, n, F, k0, rs, sc, err);
    rle_expand_kernel<uint32_t><<<tiles, kThreads, 0, st>>>(in, static_cast<uint32_t*>(out), n, F, tpf, k0, rs, sc, err);
  } else {
    timing_kernel_start(st);
    rle_dscan_kernel<uint16_t><<<k1 - k0, 1024, 0, st>>>(in, n, F, k0, rs, sc, err);
    rle_expand_kernel<uint16_t><<<tiles, kThreads, 0, st>>>(in, static_cast<uint16_t*>(out), n, F, tpf, k0, rs, sc, err);
  }
  e = cudaGetLastError();
  cudaFreeAsync(rs, st);
  return e;
}

}  // namespace cswap
