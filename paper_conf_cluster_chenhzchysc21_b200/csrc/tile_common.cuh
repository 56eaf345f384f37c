// tile_common.cuh — shared pieces of the multi-pass codecs (RLE, CSR): tile geometry, block
// reductions / scans, tile staging.
#pragma once
#include "common.cuh"

namespace cswap {

template <typename T>
struct TileGeom {
  static constexpr int W = sizeof(T);
  static constexpr int TILE = kTileBytes / W;  // elements per tile
  static constexpr int PER_WARP = TILE / kWarps;
  static constexpr int ROWS = PER_WARP / 32;   // rows of 32 elements per warp
};

// tile t of a tensor with frames of F elements: frame k, index j in frame, start and length
struct TilePos {
  uint32_t k, j;
  uint64_t Fk, tin;
  uint32_t te;
};
template <typename T>
__device__ __forceinline__ TilePos tile_pos(uint32_t t, uint64_t n, uint64_t F, uint32_t tpf) {
  TilePos p;
  p.k = t / tpf;
  p.j = t % tpf;
  p.Fk = frame_len(n, F, p.k);
  p.tin = uint64_t(p.j) * TileGeom<T>::TILE;
  p.te = uint32_t(umin64(TileGeom<T>::TILE, p.Fk - p.tin));
  return p;
}

// Copy te elements from global (16-byte aligned start) into shared memory (16-byte vectors,
// scalar tail); zero the rest of the tile.
template <typename T>
__device__ __forceinline__ void stage_tile(T* s_x, const T* g, uint32_t te) {
  using G = TileGeom<T>;
  constexpr int EPV = 16 / sizeof(T);
  const uint32_t nv = te / EPV;
  for (uint32_t v = threadIdx.x; v < G::TILE / EPV; v += blockDim.x) {
    uint4 x = make_uint4(0, 0, 0, 0);
    if (v < nv) x = ldg_stream(reinterpret_cast<const uint4*>(g) + v);
    reinterpret_cast<uint4*>(s_x)[v] = x;
  }
  __syncthreads();
  for (uint32_t e = nv * EPV + threadIdx.x; e < te; e += blockDim.x) s_x[e] = g[e];
  __syncthreads();
}

__device__ __forceinline__ uint32_t block_sum_u32(uint32_t v, uint32_t* s_tmp /* >= 33 */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  v = __reduce_add_sync(0xffffffffu, v);
  if (lane == 0) s_tmp[warp] = v;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t a = 0;
    for (int w = 0; w < int(blockDim.x / 32); w++) a += s_tmp[w];
    s_tmp[32] = a;
  }
  __syncthreads();
  const uint32_t r = s_tmp[32];
  __syncthreads();
  return r;
}

__device__ __forceinline__ uint64_t block_min_u64(uint64_t v, uint64_t* s_tmp /* >= 33 */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t y = __shfl_xor_sync(0xffffffffu, v, o);
    v = y < v ? y : v;
  }
  if (lane == 0) s_tmp[warp] = v;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t a = ~uint64_t(0);
    for (int w = 0; w < int(blockDim.x / 32); w++) a = s_tmp[w] < a ? s_tmp[w] : a;
    s_tmp[32] = a;
  }
  __syncthreads();
  const uint64_t r = s_tmp[32];
  __syncthreads();
  return r;
}

// Block-wide exclusive prefix sum (u64) with the block total; blockDim.x <= 1024.
__device__ __forceinline__ uint64_t block_excl_sum_u64(uint64_t v, uint64_t* s_tmp /* >= 33 */, uint64_t* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t inc = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) s_tmp[warp] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t a = 0;
    for (int w = 0; w < int(blockDim.x / 32); w++) {
      const uint64_t x = s_tmp[w];
      s_tmp[w] = a;
      a += x;
    }
    s_tmp[32] = a;
  }
  __syncthreads();
  const uint64_t r = s_tmp[warp] + inc - v;
  *total = s_tmp[32];
  __syncthreads();
  return r;
}

// Block-wide exclusive prefix MIN taken from the right (suffix): r = min(v of threads > tid).
__device__ __forceinline__ uint64_t block_excl_suffix_min_u64(uint64_t v, uint64_t* s_tmp, uint64_t* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  uint64_t inc = v;  // inclusive suffix min within the warp
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_down_sync(0xffffffffu, inc, o);
    if (lane + o < 32) inc = y < inc ? y : inc;
  }
  const uint64_t after_in_warp = __shfl_down_sync(0xffffffffu, inc, 1);
  if (lane == 0) s_tmp[warp] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t a = ~uint64_t(0);
    for (int w = nw - 1; w >= 0; w--) {
      const uint64_t x = s_tmp[w];
      s_tmp[w] = a;  // min over warps after w
      a = x < a ? x : a;
    }
    s_tmp[32] = a;
  }
  __syncthreads();
  uint64_t r = s_tmp[warp];
  if (lane < 31) r = after_in_warp < r ? after_in_warp : r;
  *total = s_tmp[32];
  __syncthreads();
  return r;
}

}  // namespace cswap
