// zvc.cu — zero-value compression (ZVC) for sm_100a.
//
// PAPER.md:222 (§IV-E): "Similar to CSR, ZVC stores a float sequence as non-zero values and
// additional indexes ... it utilizes a 32-bit bitmap as the index for 32 consecutive floats".
// Byte layout: DESIGN.md §3 (frame = u32 bitmap[ceil(Fk/32)] pad16 | non-zero words pad16).
//
// Compress: ONE pass over the input.  Each CTA takes a 32 KiB tile in ticket order, builds the
// tile's bitmap words from warp shuffles of per-lane nibbles, counts non-zeros, publishes its
// byte count (decoupled lookback), learns the absolute container offset of its
// values, compacts them in shared memory at the destination's 16-byte phase and writes them with
// 128-bit stores.  Frame k's first tile chains on frame k-1's last tile to place the frame.
// Decompress: a one-CTA prep kernel validates the header and scans the frame table; then each
// CTA reads its 1 KiB bitmap slice, popcounts it, gets its in-frame value offset by lookback,
// pulls its value span into shared memory with one cp.async.bulk (TMA 1-D) and expands it
// with 128-bit stores.
#include "common.cuh"
#include "kernels.h"

namespace cswap {

template <typename T>
struct ZvcGeom {
  static constexpr int W = sizeof(T);
  static constexpr int EPV = 16 / W;                  // elements per 16-byte vector
  static constexpr int TILE = kTileBytes / W;         // elements per tile
  static constexpr int WT = TILE / 32;                // bitmap words per tile
  static constexpr int CHUNK = 32 * EPV;              // elements per warp-wide vector load
  static constexpr int PER_WARP = TILE / kWarps;      // elements per warp
  static constexpr int NCH = PER_WARP / CHUNK;        // vector loads per thread
  static constexpr int LPW = 32 / EPV;                // lanes per bitmap word
  static_assert(NCH * CHUNK * kWarps == TILE, "tile geometry");
};

__device__ __forceinline__ uint32_t nib_of(uint4 v, int /*W=4*/, uint32_t /*tag*/) {
  return (v.x != 0) | ((v.y != 0) << 1) | ((v.z != 0) << 2) | ((v.w != 0) << 3);
}
__device__ __forceinline__ uint32_t nib16(uint4 v) {
  auto h = [](uint32_t u) { return ((u & 0xFFFFu) != 0) | (((u >> 16) != 0) << 1); };
  return h(v.x) | (h(v.y) << 2) | (h(v.z) << 4) | (h(v.w) << 6);
}
template <typename T>
__device__ __forceinline__ uint32_t nonzero_bits(uint4 v) {
  if constexpr (sizeof(T) == 4) return nib_of(v, 4, 0);
  else return nib16(v);
}
template <typename T>
__device__ __forceinline__ uint32_t lane_elem(const uint4& v, int i) {
  const uint32_t w[4] = {v.x, v.y, v.z, v.w};
  if constexpr (sizeof(T) == 4) return w[i];
  else return (w[i >> 1] >> ((i & 1) * 16)) & 0xFFFFu;
}

// ------------------------------------------------------------------------------------------
template <typename T>
__global__ void __launch_bounds__(kThreads, 4)
    zvc_compress_kernel(const T* __restrict__ in, uint64_t n, uint64_t F, uint32_t K, uint32_t tpf,
                        uint32_t num_tiles, uint8_t* __restrict__ out, uint64_t* out_size, Scratch sc,
                        uint32_t epoch, int dtype) {
  using G = ZvcGeom<T>;
  __shared__ uint32_t s_ticket;
  __shared__ uint32_t s_warp_off[kWarps + 1];
  __shared__ uint64_t s_excl, s_fstart;
  __shared__ __align__(16) uint32_t s_bm[G::WT];
  extern __shared__ __align__(16) uint8_t s_out[];  // kTileBytes + 16

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) s_ticket = atomicAdd(sc.tickets + epoch, 1u);
  __syncthreads();
  const uint32_t t = s_ticket;
  const uint32_t k = t / tpf, j = t % tpf;
  const uint64_t Fk = frame_len(n, F, k);
  const uint64_t tin = uint64_t(j) * G::TILE;  // tile start inside the frame
  const uint32_t tile_elems = uint32_t(umin64(G::TILE, Fk - tin));
  const T* src = in + uint64_t(k) * F + tin;
  const bool last_in_frame = tin + G::TILE >= Fk;

  // ---- 1. load, bitmap words, counts ----------------------------------------------------
  uint4 v[G::NCH];
  uint32_t bits[G::NCH];
  uint32_t pos[G::NCH];  // in-warp exclusive rank of this lane's first element, per chunk
  uint32_t warp_total = 0;
#pragma unroll
  for (int q = 0; q < G::NCH; q++) {
    const uint32_t e0 = warp * G::PER_WARP + q * G::CHUNK + lane * G::EPV;
    if (e0 + G::EPV <= tile_elems) {
      v[q] = ldg_stream(reinterpret_cast<const uint4*>(src + e0));
    } else {
      uint32_t w4[4] = {0, 0, 0, 0};
      for (int i = 0; i < G::EPV; i++)
        if (e0 + i < tile_elems) {
          uint32_t x = uint32_t(src[e0 + i]);
          if constexpr (sizeof(T) == 4) w4[i] = x;
          else w4[i >> 1] |= x << ((i & 1) * 16);
        }
      v[q] = make_uint4(w4[0], w4[1], w4[2], w4[3]);
    }
  }
#pragma unroll
  for (int q = 0; q < G::NCH; q++) {
    const uint32_t b = nonzero_bits<T>(v[q]);
    bits[q] = b;
    // bitmap word = OR of the LPW lanes' bit groups, each shifted to its element position
    uint32_t word = b << ((lane % G::LPW) * G::EPV);
    word |= __shfl_xor_sync(0xffffffffu, word, 1);
    word |= __shfl_xor_sync(0xffffffffu, word, 2);
    if (G::LPW >= 8) word |= __shfl_xor_sync(0xffffffffu, word, 4);
    if (lane % G::LPW == 0) s_bm[(warp * G::PER_WARP + q * G::CHUNK) / 32 + lane / G::LPW] = word;
    // inclusive warp scan of per-lane counts
    const uint32_t c = __popc(b);
    uint32_t inc = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
    pos[q] = warp_total + inc - c;
    warp_total += __shfl_sync(0xffffffffu, inc, 31);
  }
  if (lane == 0) s_warp_off[warp + 1] = warp_total;
  __syncthreads();
  if (tid == 0) {
    uint32_t acc = 0;
    s_warp_off[0] = 0;
    for (int w = 0; w < kWarps; w++) {
      acc += s_warp_off[w + 1];
      s_warp_off[w + 1] = acc;
    }
  }
  __syncthreads();
  const uint32_t tile_nnz = s_warp_off[kWarps];
  const uint64_t tile_bytes = uint64_t(tile_nnz) * G::W;

  // ---- 2. publish aggregate, look back, publish inclusive prefix --------------------------
  const uint64_t nwords_k = cdiv(Fk, 32);
  if (warp == 0) {
    if (j > 0 && lane == 0) st_release(sc.status + t, make_status(tile_bytes, epoch, kFlagA));
    uint64_t excl, fstart;
    if (j == 0) {
      if (lane == 0) {
        if (k == 0) {
          fstart = data_start(K);
        } else {
          uint64_t s;
          do { s = ld_acquire(sc.status + t - 1); } while (status_flag(s, epoch) != kFlagP);
          fstart = a16(status_value(s));
        }
        excl = fstart + a16(4 * nwords_k);
        st_release(sc.aux + k, fstart);
        st_release(sc.status + t, make_status(excl + tile_bytes, epoch, kFlagP));
        s_excl = excl;
        s_fstart = fstart;
      }
    } else {
      excl = lookback(sc.status, t, int64_t(t) - j, epoch);
      if (lane == 0) {
        st_release(sc.status + t, make_status(excl + tile_bytes, epoch, kFlagP));
        s_excl = excl;
        s_fstart = ld_acquire(sc.aux + k);
      }
    }
  }
  __syncthreads();
  const uint64_t g0 = s_excl, fstart = s_fstart;
  const uint32_t d = uint32_t(g0 & 15);

  // ---- 3. compact into shared memory at the destination's 16-byte phase ------------------
  const uint32_t woff = s_warp_off[warp];
#pragma unroll
  for (int q = 0; q < G::NCH; q++) {
    uint32_t b = bits[q];
    uint32_t r = woff + pos[q];
#pragma unroll
    for (int i = 0; i < G::EPV; i++) {
      if (b & (1u << i)) {
        const uint32_t x = lane_elem<T>(v[q], i);
        if constexpr (sizeof(T) == 4) *reinterpret_cast<uint32_t*>(s_out + d + 4 * r) = x;
        else *reinterpret_cast<uint16_t*>(s_out + d + 2 * r) = uint16_t(x);
        r++;
      }
    }
  }
  __syncthreads();

  // ---- 4. stores: values (16-byte vectors, element-wise head/tail), bitmap, frame pad -----
  uint8_t* gdst = out + (g0 - d);
  const uint32_t span = d + uint32_t(tile_bytes);
  const uint32_t nvec = (span + 15) / 16;
  for (uint32_t c = tid; c < nvec; c += kThreads) {
    const uint32_t lo = 16 * c, hi = lo + 16;
    if (lo >= d && hi <= span) {
      stg_stream(reinterpret_cast<uint4*>(gdst + lo), *reinterpret_cast<const uint4*>(s_out + lo));
    } else {
      for (uint32_t b = max(lo, d); b < min(hi, span); b += G::W) {
        if constexpr (sizeof(T) == 4) *reinterpret_cast<uint32_t*>(gdst + b) = *reinterpret_cast<const uint32_t*>(s_out + b);
        else *reinterpret_cast<uint16_t*>(gdst + b) = *reinterpret_cast<const uint16_t*>(s_out + b);
      }
    }
  }
  const uint64_t g1 = g0 + tile_bytes;
  if (last_in_frame && tid == kThreads - 1) {
    for (uint64_t b = g1; b < a16(g1); b += 2) *reinterpret_cast<uint16_t*>(out + b) = 0;
    *reinterpret_cast<uint64_t*>(out + 64 + 8ull * k) = a16(g1) - fstart;  // frame_bytes[k]
  }
  {
    const uint64_t w0 = uint64_t(j) * G::WT;
    const uint64_t wend = last_in_frame ? ((nwords_k + 3) & ~uint64_t(3)) : w0 + G::WT;
    const uint32_t nv = uint32_t((wend - w0) / 4);
    uint4* bdst = reinterpret_cast<uint4*>(out + fstart + 4 * w0);
    for (uint32_t c = tid; c < nv; c += kThreads) stg_stream(bdst + c, reinterpret_cast<const uint4*>(s_bm)[c]);
  }
  if (t == num_tiles - 1 && tid == 0) {
    const uint64_t total = a16(g1);
    write_header(out, kZVC, dtype, n, F, K, 0, total);
    for (uint64_t b = 64 + 8ull * K; b < data_start(K); b += 8) *reinterpret_cast<uint64_t*>(out + b) = 0;
    *out_size = total;
  }
}

// ------------------------------------------------------------------------------------------
template <typename T>
__global__ void __launch_bounds__(kThreads, 4)
    zvc_decompress_kernel(const uint8_t* __restrict__ in, T* __restrict__ outp, uint64_t n, uint64_t F,
                          uint32_t K, uint32_t tpf, uint32_t k0, uint32_t num_tiles, Scratch sc, uint32_t epoch,
                          uint32_t* err) {
  using G = ZvcGeom<T>;
  __shared__ uint32_t s_ticket;
  __shared__ uint32_t s_warp_off[kWarps + 1];
  __shared__ uint64_t s_excl;
  __shared__ __align__(8) uint64_t s_bar;
  __shared__ __align__(16) uint32_t s_bm[G::WT];
  extern __shared__ __align__(16) uint8_t s_val[];  // kTileBytes + 32

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (*reinterpret_cast<volatile uint32_t*>(err) != 0) return;  // header rejected by prep
  if (tid == 0) s_ticket = atomicAdd(sc.tickets + epoch, 1u);
  __syncthreads();
  const uint32_t t = s_ticket + k0 * tpf;  // status index (frame-major)
  const uint32_t k = t / tpf, j = t % tpf;
  const uint64_t Fk = frame_len(n, F, k);
  const uint64_t tin = uint64_t(j) * G::TILE;
  const uint32_t tile_elems = uint32_t(umin64(G::TILE, Fk - tin));
  const uint64_t fstart = sc.aux[k];
  const uint64_t fbytes = sc.aux2[k];
  const uint64_t nwords_k = cdiv(Fk, 32);
  const uint64_t bm_bytes = a16(4 * nwords_k);
  const bool last_in_frame = tin + G::TILE >= Fk;
  bool bad = bm_bytes > fbytes;

  // ---- 1. bitmap slice -> smem; counts ---------------------------------------------------
  const uint32_t nw_tile = uint32_t(cdiv(tile_elems, 32));
  {
    const uint32_t* bsrc = reinterpret_cast<const uint32_t*>(in + fstart) + uint64_t(j) * G::WT;
    const uint32_t nv = (nw_tile + 3) / 4;
    for (uint32_t c = tid; c < G::WT / 4; c += kThreads) {
      uint4 x = make_uint4(0, 0, 0, 0);
      if (c < nv && !bad) x = *reinterpret_cast<const uint4*>(bsrc + 4 * c);
      reinterpret_cast<uint4*>(s_bm)[c] = x;
    }
  }
  if (tid == 0) mbar_init(&s_bar, 1);
  __syncthreads();
  if (tid == 0 && (tile_elems & 31)) {  // bits past the frame end must be zero
    uint32_t& last = s_bm[nw_tile - 1];
    if (last >> (tile_elems & 31)) { bad = true; last &= (1u << (tile_elems & 31)) - 1; }
  }
  if (bad) set_error(err, kErrCorrupt);
  __syncthreads();
  uint32_t wt = 0;
  {
    constexpr int WPW = G::WT / kWarps;  // words per warp (32 or 64)
#pragma unroll
    for (int i = 0; i < WPW / 32; i++) wt += __popc(s_bm[warp * WPW + i * 32 + lane]);
    wt = __reduce_add_sync(0xffffffffu, wt);
  }
  if (lane == 0) s_warp_off[warp + 1] = wt;
  __syncthreads();
  if (tid == 0) {
    uint32_t acc = 0;
    s_warp_off[0] = 0;
    for (int w = 0; w < kWarps; w++) {
      acc += s_warp_off[w + 1];
      s_warp_off[w + 1] = acc;
    }
  }
  __syncthreads();
  const uint32_t tile_nnz = s_warp_off[kWarps];

  // ---- 2. in-frame popcount prefix by lookback ------------------------------------------
  if (warp == 0) {
    uint64_t excl = 0;
    if (j > 0) {
      if (lane == 0) st_release(sc.status + t, make_status(tile_nnz, epoch, kFlagA));
      excl = lookback(sc.status, t, int64_t(t) - j, epoch);
    }
    if (lane == 0) {
      st_release(sc.status + t, make_status(excl + tile_nnz, epoch, kFlagP));
      s_excl = excl;
      if (last_in_frame && bm_bytes + a16(G::W * (excl + tile_nnz)) != fbytes) set_error(err, kErrCorrupt);
    }
  }
  __syncthreads();
  const uint64_t excl = s_excl;

  // ---- 3. value span -> smem with one bulk copy (aligned superset) ----------------------
  const uint64_t vbeg = fstart + bm_bytes + uint64_t(G::W) * excl;
  const uint64_t vend = vbeg + uint64_t(G::W) * tile_nnz;
  const uint64_t abeg = vbeg & ~uint64_t(15), aend = a16(vend);
  const uint32_t d = uint32_t(vbeg - abeg);
  const bool in_bounds = aend <= fstart + fbytes;
  if (!in_bounds && tid == 0) set_error(err, kErrCorrupt);
  if (tid == 0) {
    const uint32_t bytes = in_bounds ? uint32_t(aend - abeg) : 0;
    if (bytes) {
      mbar_expect_tx(&s_bar, bytes);
      bulk_g2s(s_val, in + abeg, bytes, &s_bar);
    } else {
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(
                       static_cast<uint32_t>(__cvta_generic_to_shared(&s_bar)))
                   : "memory");
    }
  }
  mbar_wait(&s_bar, 0);

  // ---- 4. expand: each lane rebuilds EPV elements -> one 16-byte store --------------------
  T* dst = outp + uint64_t(k) * F + tin;
  uint32_t r = s_warp_off[warp];
#pragma unroll
  for (int q = 0; q < G::NCH; q++) {
    const uint32_t e0 = warp * G::PER_WARP + q * G::CHUNK + lane * G::EPV;
    const uint32_t wbase = e0 / 32;  // first bitmap word of this chunk is (chunk start)/32
    const uint32_t cw0 = (warp * G::PER_WARP + q * G::CHUNK) / 32;
    uint32_t before = 0, mine = 0;
#pragma unroll
    for (int m = 0; m < G::EPV; m++) {  // the EPV words of this chunk
      const uint32_t wd = s_bm[cw0 + m];
      if (cw0 + m < wbase) before += __popc(wd);
      if (cw0 + m == wbase) mine = wd;
    }
    const uint32_t sh = (lane % G::LPW) * G::EPV;
    const uint32_t b = (mine >> sh) & ((1u << G::EPV) - 1);
    uint32_t rank = r + before + __popc(mine & ((1u << sh) - 1));
    uint32_t w4[4] = {0, 0, 0, 0};
#pragma unroll
    for (int i = 0; i < G::EPV; i++) {
      if (b & (1u << i)) {
        uint32_t x;
        if constexpr (sizeof(T) == 4) x = *reinterpret_cast<const uint32_t*>(s_val + d + 4 * rank);
        else x = *reinterpret_cast<const uint16_t*>(s_val + d + 2 * rank);
        if constexpr (sizeof(T) == 4) w4[i] = x;
        else w4[i >> 1] |= x << ((i & 1) * 16);
        rank++;
      }
    }
    uint32_t chunk_total = 0;
#pragma unroll
    for (int m = 0; m < G::EPV; m++) chunk_total += __popc(s_bm[cw0 + m]);
    r += chunk_total;
    if (!in_bounds) w4[0] = w4[1] = w4[2] = w4[3] = 0;
    if (e0 + G::EPV <= tile_elems) {
      stg_stream(reinterpret_cast<uint4*>(dst + e0), make_uint4(w4[0], w4[1], w4[2], w4[3]));
    } else {
      for (int i = 0; i < G::EPV; i++)
        if (e0 + i < tile_elems) {
          if constexpr (sizeof(T) == 4) dst[e0 + i] = w4[i];
          else dst[e0 + i] = T((w4[i >> 1] >> ((i & 1) * 16)) & 0xFFFFu);
        }
    }
  }
}

// ------------------------------------------------------------------------------------------
template <typename T>
static cudaError_t launch_zvc_compress_t(const void* in, uint64_t n, uint64_t F, uint8_t* out, uint64_t* out_size,
                                         const Scratch& sc, uint32_t epoch, int dtype, cudaStream_t st) {
  using G = ZvcGeom<T>;
  const uint32_t K = uint32_t(cdiv(n, F));
  const uint32_t tpf = uint32_t(cdiv(F, G::TILE));
  const uint32_t tiles = (K - 1) * tpf + uint32_t(cdiv(frame_len(n, F, K - 1), G::TILE));
  const int smem = kTileBytes + 16;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(zvc_compress_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  zvc_compress_kernel<T><<<tiles, kThreads, smem, st>>>(static_cast<const T*>(in), n, F, K, tpf, tiles, out,
                                                        out_size, sc, epoch, dtype);
  return cudaGetLastError();
}

cudaError_t launch_zvc_compress(const void* in, uint64_t n, int w, uint64_t F, uint8_t* out, uint64_t* out_size,
                                const Scratch& sc, uint32_t epoch, int dtype, cudaStream_t st) {
  return w == 4 ? launch_zvc_compress_t<uint32_t>(in, n, F, out, out_size, sc, epoch, dtype, st)
                : launch_zvc_compress_t<uint16_t>(in, n, F, out, out_size, sc, epoch, dtype, st);
}

uint32_t zvc_tiles(uint64_t n, int w, uint64_t F, uint32_t k0, uint32_t k1, uint32_t* tpf_out) {
  const uint32_t TILE = kTileBytes / w;
  const uint32_t tpf = uint32_t(cdiv(F, TILE));
  if (tpf_out) *tpf_out = tpf;
  if (k1 <= k0) return 0;
  return (k1 - 1 - k0) * tpf + uint32_t(cdiv(frame_len(n, F, k1 - 1), TILE));
}

template <typename T>
static cudaError_t launch_zvc_decompress_t(const uint8_t* in, void* out, uint64_t n, uint64_t F, uint32_t k0,
                                           uint32_t k1, const Scratch& sc, uint32_t epoch, uint32_t* err,
                                           cudaStream_t st) {
  const uint32_t K = uint32_t(cdiv(n, F));
  uint32_t tpf;
  const uint32_t tiles = zvc_tiles(n, sizeof(T), F, k0, k1, &tpf);
  if (!tiles) return cudaSuccess;
  const int smem = kTileBytes + 32;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(zvc_decompress_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  zvc_decompress_kernel<T><<<tiles, kThreads, smem, st>>>(in, static_cast<T*>(out), n, F, K, tpf, k0, tiles, sc,
                                                          epoch, err);
  return cudaGetLastError();
}

cudaError_t launch_zvc_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t k0,
                                  uint32_t k1, const Scratch& sc, uint32_t epoch, uint32_t* err, cudaStream_t st) {
  return w == 4 ? launch_zvc_decompress_t<uint32_t>(in, out, n, F, k0, k1, sc, epoch, err, st)
                : launch_zvc_decompress_t<uint16_t>(in, out, n, F, k0, k1, sc, epoch, err, st);
}

}  // namespace cswap
