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
// Decompress: chunked scan of the lengths (chunk sums -> per-frame scan of the chunk sums), then
// run-parallel expansion (see rle_runs_kernel).
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
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
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
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
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
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
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
  __shared__ uint32_t s_wfirst[kWarps], s_wnext[kWarps];
  __syncwarp();
  if (lane == 0) {
    s_wcnt[warp] = cnt;
    s_wfirst[warp] = cnt ? uint32_t(wpos[0]) : 0xFFFFFFFFu;
  }
  __syncthreads();
  if (tid == 0) {  // run offset of each warp's list, and the first run start after each warp
    uint32_t a = 0, nx = 0xFFFFFFFFu;
    for (int w = kWarps - 1; w >= 0; w--) {
      s_wnext[w] = nx;
      if (s_wfirst[w] != 0xFFFFFFFFu) nx = s_wfirst[w];
    }
    for (int w = 0; w < kWarps; w++) {
      const uint32_t x = s_wcnt[w];
      s_wcnt[w] = a;
      a += x;
    }
    s_wcnt[kWarps] = a;
  }
  __syncthreads();
  const uint64_t run_off = sc.tbuf[t];
  const uint64_t next_start = sc.tbuf2[t];
  const uint64_t r_k = sc.aux3[p.k];
  const uint64_t fstart = sc.aux[p.k];
  uint32_t* lengths = reinterpret_cast<uint32_t*>(out + fstart + 16) + run_off + s_wcnt[warp];
  T* values = reinterpret_cast<T*>(out + fstart + 16 + a16(4 * r_k)) + run_off + s_wcnt[warp];
  // each warp writes the runs starting in its slab: consecutive lanes, consecutive runs
  const uint64_t after = s_wnext[warp] != 0xFFFFFFFFu ? p.tin + s_wnext[warp] : next_start;
  for (uint32_t q = lane; q < cnt; q += 32) {
    const uint32_t pos = wpos[q];
    const uint64_t end = q + 1 < cnt ? p.tin + wpos[q + 1] : after;
    lengths[q] = uint32_t(end - (p.tin + pos));
    values[q] = s_x[pos];
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
  CUDA_TRY_LAUNCH(pdl_launch(rle_count_kernel<T>, dim3(tiles), dim3(kThreads), 0, st, x, n, F, tpf, sc));
  CUDA_TRY_LAUNCH(pdl_launch(rle_scan_kernel<T>, dim3(K), dim3(1024), 0, st, n, F, tpf, sc));
  cudaError_t e = launch_finalize(out, kRLE, dtype, n, F, 0, sc, out_size, st);
  if (e != cudaSuccess) return e;
  const int smem = G::TILE * 2;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(rle_emit_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  CUDA_TRY_LAUNCH(pdl_launch(rle_emit_kernel<T>, dim3(tiles), dim3(kThreads), smem, st, x, n, F, tpf, out, sc));
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
// ---- decompress ------------------------------------------------------------------------------
// The lengths of frame k are cut into chunks of kRleChunk runs.  (1) one warp per chunk slot sums
// its chunk's lengths; (2) one CTA per frame validates the frame and scans the chunk sums into
// chunk start positions; (3) rle_runs_kernel expands the runs of each chunk straight into the
// output (run-parallel; long runs go to a piece list); (4) rle_fill_kernel fills the pieces.
// Traffic: lengths twice, values once, output once.
constexpr uint32_t kRleChunk = 1024;

__device__ __forceinline__ bool rle_frame_header(const uint8_t* in, uint64_t fstart, uint64_t fb, uint64_t Fk, int w,
                                                 uint64_t* r_out) {
  if (fb < 16) return false;
  const uint64_t r = *reinterpret_cast<const uint32_t*>(in + fstart);
  *r_out = r;
  return r >= 1 && r <= Fk && fb == 16 + a16(4 * r) + a16(uint64_t(w) * r);
}

// one warp per chunk slot, grid-stride (most slots of a frame are empty when runs are long)
__global__ void __launch_bounds__(kThreads) rle_dsum_kernel(const uint8_t* __restrict__ in, uint64_t n, uint64_t F,
                                                            int w, uint32_t k0, uint32_t k1, uint32_t cpf,
                                                            uint64_t* csum, uint32_t* npieces, Scratch sc,
                                                            uint32_t* err) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  if (blockIdx.x == 0 && threadIdx.x == 0) *npieces = 0;  // rle_runs_kernel appends long-run pieces
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const int lane = threadIdx.x & 31;
  const uint64_t slots = uint64_t(k1 - k0) * cpf;
  const uint64_t nwarps = uint64_t(gridDim.x) * kWarps;
  for (uint64_t sl = uint64_t(blockIdx.x) * kWarps + (threadIdx.x >> 5); sl < slots; sl += nwarps) {
    const uint32_t k = k0 + uint32_t(sl / cpf), c = uint32_t(sl % cpf);
    const uint64_t Fk = frame_len(n, F, k);
    uint64_t r;
    if (!rle_frame_header(in, sc.aux[k], sc.aux2[k], Fk, w, &r)) continue;  // flagged by rle_dscan2
    const uint64_t i0 = uint64_t(c) * kRleChunk;
    if (i0 >= r) {  // past the frame's last chunk: skip the rest of this frame's slots
      continue;
    }
    const uint32_t m = uint32_t(umin64(kRleChunk, r - i0));
    const uint32_t* len = reinterpret_cast<const uint32_t*>(in + sc.aux[k] + 16) + i0;
    uint64_t acc = 0;  // <= kRleChunk * 2^32
    bool zero = false;
#pragma unroll 8
    for (uint32_t i = lane; i < m; i += 32) {
      const uint32_t v = len[i];
      zero |= v == 0;
      acc += v;
    }
    if (__any_sync(0xffffffffu, zero) && lane == 0) set_error(err, kErrCorrupt);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) csum[sl] = acc;
  }
}

__global__ void __launch_bounds__(1024) rle_dscan2_kernel(const uint8_t* __restrict__ in, uint64_t n, uint64_t F,
                                                          int w, uint32_t k0, uint32_t cpf, uint64_t* csum,
                                                          Scratch sc, uint32_t* err) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  __shared__ uint64_t s_tmp[33];
  __shared__ int s_ok;
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const uint32_t k = k0 + blockIdx.x;
  const uint64_t Fk = frame_len(n, F, k);
  if (threadIdx.x == 0) {
    uint64_t r = 0;
    const bool ok = rle_frame_header(in, sc.aux[k], sc.aux2[k], Fk, w, &r);
    sc.aux3[k] = ok ? r : 0;
    s_ok = ok;
    if (!ok) set_error(err, kErrCorrupt);
  }
  __syncthreads();
  if (!s_ok) return;
  const uint32_t nch = uint32_t(cdiv(sc.aux3[k], kRleChunk));
  uint64_t* cs = csum + uint64_t(blockIdx.x) * cpf;
  uint64_t carry = 0;
  for (uint32_t c0 = 0; c0 < nch; c0 += blockDim.x) {
    const uint32_t c = c0 + threadIdx.x;
    const uint64_t v = c < nch ? cs[c] : 0;
    uint64_t tot;
    const uint64_t ex = block_excl_sum_u64(v, s_tmp, &tot);
    if (c < nch) cs[c] = carry + ex;  // chunk start position inside the frame
    carry += tot;
  }
  if (threadIdx.x == 0 && carry != Fk) set_error(err, kErrCorrupt);
}

// Run-parallel expansion: one CTA per chunk slot (grid-stride), 8 warps x 128 consecutive runs.
// Lane l of a warp holds runs l, 32+l, 64+l, 96+l, so one store instruction writes 32
// consecutive runs' elements (coalesced for the short runs that dominate iid ReLU data).  Runs of
// 33..kLongRun elements are filled by the whole warp; longer runs are cut into kPiece-element
// pieces appended to a global list that rle_fill_kernel spreads over the grid (one run may
// cover a whole frame).
constexpr uint32_t kLongRun = 4096, kPiece = 8192;
struct RlePiece {
  uint64_t start;  // element index in the tensor
  uint32_t len, value;
};

template <typename T>
__global__ void __launch_bounds__(kThreads) rle_runs_kernel(const uint8_t* __restrict__ in, T* __restrict__ outp,
                                                            uint64_t n, uint64_t F, uint32_t k0, uint32_t k1,
                                                            uint32_t cpf, const uint64_t* __restrict__ cstart,
                                                            RlePiece* pieces, uint32_t* npieces, uint64_t cap,
                                                            Scratch sc, uint32_t* err) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  __shared__ uint64_t s_wtot[kWarps];
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t slots = uint64_t(k1 - k0) * cpf;
  for (uint64_t sl = blockIdx.x; sl < slots; sl += gridDim.x) {
    const uint32_t k = k0 + uint32_t(sl / cpf), c = uint32_t(sl % cpf);
    const uint64_t r = sc.aux3[k];  // validated by rle_dscan2 (0: corrupt frame)
    const uint64_t i0 = uint64_t(c) * kRleChunk;
    if (i0 >= r) continue;  // uniform over the CTA
    const uint32_t m = uint32_t(umin64(kRleChunk, r - i0));
    const uint32_t* lens = reinterpret_cast<const uint32_t*>(in + sc.aux[k] + 16) + i0;
    const T* vals = reinterpret_cast<const T*>(in + sc.aux[k] + 16 + a16(4 * r)) + i0;
    const uint32_t wb = warp * (kRleChunk / kWarps);
    constexpr int Q = kRleChunk / kWarps / 32;
    uint32_t L[Q];
    T V[Q];
    uint64_t S[Q], carry = 0;
#pragma unroll
    for (int q = 0; q < Q; q++) {
      const uint32_t i = wb + q * 32 + lane;
      L[q] = i < m ? lens[i] : 0u;
      V[q] = i < m ? vals[i] : T(0);
    }
#pragma unroll
    for (int q = 0; q < Q; q++) {  // exclusive prefix of the warp's runs, in run order
      uint64_t inc = L[q];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
      }
      S[q] = carry + inc - L[q];
      carry += __shfl_sync(0xffffffffu, inc, 31);
    }
    if (lane == 0) s_wtot[warp] = carry;
    __syncthreads();
    uint64_t wbase = cstart[sl];
    for (int q = 0; q < warp; q++) wbase += s_wtot[q];
    T* dst = outp + uint64_t(k) * F;
#pragma unroll
    for (int q = 0; q < Q; q++) {
      const uint64_t st = wbase + S[q];
      const uint32_t len = L[q];
      const uint32_t sh = len <= 32 ? len : 0u;
      const uint32_t mx = __reduce_max_sync(0xffffffffu, sh);
      for (uint32_t e = 0; e < mx; e++)
        if (e < sh) dst[st + e] = V[q];
      uint32_t med = __ballot_sync(0xffffffffu, len > 32 && len <= kLongRun);
      while (med) {
        const int b = __ffs(med) - 1;
        med &= med - 1;
        const uint64_t s2 = __shfl_sync(0xffffffffu, st, b);
        const uint32_t l2 = __shfl_sync(0xffffffffu, len, b);
        const T v2 = T(__shfl_sync(0xffffffffu, uint32_t(V[q]), b));
        for (uint32_t x = lane; x < l2; x += 32) dst[s2 + x] = v2;
      }
      if (len > kLongRun) {
        const uint32_t np = (len + kPiece - 1) / kPiece;
        const uint32_t idx = atomicAdd(npieces, np);
        if (uint64_t(idx) + np > cap) {
          set_error(err, kErrCorrupt);  // cannot happen for a valid container (cap >= n / kLongRun)
        } else {
          for (uint32_t p2 = 0; p2 < np; p2++)
            pieces[idx + p2] = RlePiece{uint64_t(k) * F + st + uint64_t(p2) * kPiece,
                                        (len - p2 * kPiece < kPiece ? len - p2 * kPiece : kPiece), uint32_t(V[q])};
        }
      }
    }
    __syncthreads();  // s_wtot is rewritten by the next slot
  }
}

template <typename T>
__global__ void __launch_bounds__(kThreads) rle_fill_kernel(T* __restrict__ outp, const RlePiece* pieces,
                                                            const uint32_t* npieces) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  const uint32_t total = *npieces;
  for (uint32_t p = blockIdx.x; p < total; p += gridDim.x) {
    const RlePiece pc = pieces[p];
    const T v = T(pc.value);
    for (uint32_t x = threadIdx.x; x < pc.len; x += blockDim.x) outp[pc.start + x] = v;
  }
}

// scratch of one decode of frames [k0, k1): chunk sums / starts | piece counter | pieces
static void rle_dtmp_layout(uint64_t n, uint64_t F, uint32_t k0, uint32_t k1, uint64_t* slots, uint64_t* cap,
                            uint64_t* off_cnt, uint64_t* off_pc, uint64_t* bytes) {
  const uint32_t cpf = uint32_t(cdiv(F, kRleChunk));  // chunk slots per frame (r_k <= F_k <= F)
  *slots = uint64_t(k1 - k0) * cpf;
  const uint64_t elems = umin64(n, uint64_t(k1) * F) - uint64_t(k0) * F;
  *cap = elems / kLongRun + (elems / kPiece) + 2 * (k1 - k0) + 8;  // pieces
  *off_cnt = a16(*slots * 8);
  *off_pc = *off_cnt + 16;
  *bytes = *off_pc + *cap * sizeof(RlePiece);
}

uint64_t rle_decompress_tmp_bytes(uint64_t n, uint64_t F, uint32_t k0, uint32_t k1) {
  if (k1 <= k0) return 0;
  uint64_t slots, cap, off_cnt, off_pc, bytes;
  rle_dtmp_layout(n, F, k0, k1, &slots, &cap, &off_cnt, &off_pc, &bytes);
  return bytes;
}

// `tmp` (rle_decompress_tmp_bytes) is owned by the caller, so the launch group allocates nothing
// and can be captured into a graph
cudaError_t launch_rle_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t k0,
                                  uint32_t k1, const Scratch& sc, uint32_t /*epoch*/, uint32_t* err, uint8_t* tmp,
                                  cudaStream_t st) {
  if (k1 <= k0) return cudaSuccess;
  const uint32_t cpf = uint32_t(cdiv(F, kRleChunk));
  uint64_t slots, cap, off_cnt, off_pc, bytes;
  rle_dtmp_layout(n, F, k0, k1, &slots, &cap, &off_cnt, &off_pc, &bytes);
  uint64_t* cs = reinterpret_cast<uint64_t*>(tmp);
  uint32_t* cnt = reinterpret_cast<uint32_t*>(tmp + off_cnt);
  RlePiece* pcs = reinterpret_cast<RlePiece*>(tmp + off_pc);
  timing_kernel_start(st);
  const uint64_t dgrid = std::min<uint64_t>(cdiv(slots, kWarps), 148 * 16);
  CUDA_TRY_LAUNCH(pdl_launch(rle_dsum_kernel, dim3(uint32_t(dgrid)), dim3(kThreads), 0, st, in, n, F, w, k0, k1, cpf, cs, cnt, sc, err));
  CUDA_TRY_LAUNCH(pdl_launch(rle_dscan2_kernel, dim3(k1 - k0), dim3(1024), 0, st, in, n, F, w, k0, cpf, cs, sc, err));
#ifndef CSWAP_RLE_RGRID
#define CSWAP_RLE_RGRID (148 * 32)  // grid-stride CTAs of the run expansion (148 * 8: 6-14 % slower)
#endif
  const uint32_t rgrid = uint32_t(CSWAP_RLE_RGRID ? std::min<uint64_t>(slots, CSWAP_RLE_RGRID) : slots);
  const uint32_t fgrid = 148 * 4;
  if (w == 4) {
    CUDA_TRY_LAUNCH(pdl_launch(rle_runs_kernel<uint32_t>, dim3(rgrid), dim3(kThreads), 0, st, in, static_cast<uint32_t*>(out), n, F, k0, k1, cpf, cs,
                                                          pcs, cnt, cap, sc, err));
    CUDA_TRY_LAUNCH(pdl_launch(rle_fill_kernel<uint32_t>, dim3(fgrid), dim3(kThreads), 0, st, static_cast<uint32_t*>(out), pcs, cnt));
  } else {
    CUDA_TRY_LAUNCH(pdl_launch(rle_runs_kernel<uint16_t>, dim3(rgrid), dim3(kThreads), 0, st, in, static_cast<uint16_t*>(out), n, F, k0, k1, cpf, cs,
                                                          pcs, cnt, cap, sc, err));
    CUDA_TRY_LAUNCH(pdl_launch(rle_fill_kernel<uint16_t>, dim3(fgrid), dim3(kThreads), 0, st, static_cast<uint16_t*>(out), pcs, cnt));
  }
  return cudaGetLastError();
}

}  // namespace cswap
