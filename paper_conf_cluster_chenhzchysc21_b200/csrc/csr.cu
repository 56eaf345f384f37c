// csr.cu — compressed sparse rows for sm_100a.
//
// PAPER.md:220 (§IV-E): "CSR compresses an original sequence as a non-zero value sequence and an
// additional index representing the locations of non-zero values. For example, a sequence
// (A00B0C000) can be compressed as (ABC) and (035)."  Reading R5: rows of C
// elements; u32 row_ptr[R+1] pad16 | u32 col_idx[nnz] pad16 | values[nnz] pad16 per frame.
//
// col_idx and values follow all row pointers / indices of the frame, so compress is count ->
// per-frame scan -> frame table -> emit (one warp per 1024-element slab, ballot ranks).
// Decompress: one CTA per output tile zero-fills the tile in shared memory, scatters the non-
// zeros of the rows it covers (column windows found by binary search), and stores the tile.
#include "kernels.h"
#include "tile_common.cuh"

namespace cswap {

// rows of 32 elements per batch of the emit pass's global loads
#ifndef CSWAP_CSR_EMIT_BATCH
#define CSWAP_CSR_EMIT_BATCH 8
#endif

template <typename T>
__global__ void __launch_bounds__(kThreads) csr_count_kernel(const T* __restrict__ in, uint64_t n, uint64_t F,
                                                             uint32_t tpf, Scratch sc) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  using G = TileGeom<T>;
  __shared__ uint32_t s_tmp[33];
  const uint32_t t = blockIdx.x;
  const TilePos p = tile_pos<T>(t, n, F, tpf);
  const T* src = in + uint64_t(p.k) * F + p.tin;
  // per-warp counts of the emit kernel's slabs (warp w: elements [w*PER_WARP, (w+1)*PER_WARP)),
  // kept in tbuf2 so that the emit pass reads the tile once
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t c = 0;
  if (p.te == G::TILE) {  // full tile: 16-byte loads, all in flight
    constexpr int V = G::TILE * int(sizeof(T)) / 16 / kThreads;
    const uint4* s4 = reinterpret_cast<const uint4*>(src) + warp * (32 * V);
    uint4 q[V];
#pragma unroll
    for (int i = 0; i < V; i++) q[i] = __ldg(s4 + lane + i * 32);
#pragma unroll
    for (int i = 0; i < V; i++) {
      if constexpr (sizeof(T) == 4) {
        c += (q[i].x != 0) + (q[i].y != 0) + (q[i].z != 0) + (q[i].w != 0);
      } else {
        const uint32_t w4[4] = {q[i].x, q[i].y, q[i].z, q[i].w};
#pragma unroll
        for (int h = 0; h < 4; h++) c += ((w4[h] & 0xFFFFu) != 0) + ((w4[h] >> 16) != 0);
      }
    }
  } else {
    const uint32_t e1 = umin32(p.te, (warp + 1) * G::PER_WARP);
    for (uint32_t e = warp * G::PER_WARP + lane; e < e1; e += 32) c += src[e] != 0;
  }
  const uint32_t wc = __reduce_add_sync(0xffffffffu, c);
  if (lane == 0) reinterpret_cast<uint32_t*>(sc.tbuf2)[uint64_t(t) * kWarps + warp] = wc;
  c = block_sum_u32(c, s_tmp);
  if (threadIdx.x == 0) sc.tbuf[t] = c;
}

// one CTA per frame: non-zero offsets per tile (tbuf), nnz_k (aux3), frame_bytes (aux2)
template <typename T>
__global__ void __launch_bounds__(1024) csr_scan_kernel(uint64_t n, uint64_t F, uint32_t tpf, uint32_t C,
                                                        Scratch sc) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  using G = TileGeom<T>;
  __shared__ uint64_t s_tmp[33];
  const uint32_t k = blockIdx.x;
  const uint64_t Fk = frame_len(n, F, k);
  const uint32_t nt = uint32_t(cdiv(Fk, G::TILE));
  uint64_t* cnt = sc.tbuf + uint64_t(k) * tpf;
  uint64_t carry = 0;
  for (uint32_t c0 = 0; c0 < nt; c0 += blockDim.x) {
    const uint32_t j = c0 + threadIdx.x;
    const uint64_t v = j < nt ? cnt[j] : 0;
    uint64_t tot;
    const uint64_t ex = block_excl_sum_u64(v, s_tmp, &tot);
    if (j < nt) cnt[j] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) {
    const uint64_t R = cdiv(Fk, C);
    sc.aux3[k] = carry;
    sc.aux2[k] = a16(4 * (R + 1)) + a16(4 * carry) + a16(uint64_t(G::W) * carry);
  }
}

template <typename T>
__global__ void __launch_bounds__(kThreads) csr_emit_kernel(const T* __restrict__ in, uint64_t n, uint64_t F,
                                                            uint32_t tpf, uint32_t C, uint8_t* __restrict__ out,
                                                            Scratch sc) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  using G = TileGeom<T>;
  __shared__ uint32_t s_wcnt[kWarps + 1];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t t = blockIdx.x;
  const TilePos p = tile_pos<T>(t, n, F, tpf);
  const T* src = in + uint64_t(p.k) * F + p.tin;
  const uint32_t lt = (1u << lane) - 1u;
  // slab offsets inside the tile from the count kernel's per-warp counts (tbuf2)
  constexpr int B = G::ROWS < CSWAP_CSR_EMIT_BATCH ? G::ROWS : CSWAP_CSR_EMIT_BATCH;
  const bool full = p.te == G::TILE;
  if (tid < kWarps) s_wcnt[tid] = reinterpret_cast<const uint32_t*>(sc.tbuf2)[uint64_t(t) * kWarps + tid];
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
  const uint64_t Fk = p.Fk, R = cdiv(Fk, C);
  const uint64_t nnz_k = sc.aux3[p.k], fstart = sc.aux[p.k];
  uint32_t* row_ptr = reinterpret_cast<uint32_t*>(out + fstart);
  uint32_t* col_idx = reinterpret_cast<uint32_t*>(out + fstart + a16(4 * (R + 1)));
  T* values = reinterpret_cast<T*>(out + fstart + a16(4 * (R + 1)) + a16(4 * nnz_k));
  const uint64_t tile_off = sc.tbuf[t];
  // pass 2: emit (col, value) at rank; row_ptr[r+1] at every row's last element
  uint64_t pre = tile_off + s_wcnt[warp];
  // column / row of tile element e: x = (tin mod C) + e; power-of-two C by mask and shift
  const uint32_t cbase = uint32_t(p.tin % C);
  const uint64_t row0 = p.tin / C;
  const bool pow2 = (C & (C - 1)) == 0;
  const int csh = __ffs(int(C)) - 1;
  // tile-local ranks (u32) against section pointers advanced to the tile's first non-zero
  uint32_t* tcol = col_idx + tile_off;
  T* tval = values + tile_off;
  uint32_t lpre = uint32_t(pre - tile_off);
  if (full && pow2 && C >= 32) {
    // fast path: a row of 32 elements never straddles a CSR row (C = 2^k >= 32 and the tile
    // starts on a multiple of 32), so its columns are colbase + lane and only lane 31 can end
    // a CSR row: per element a ballot rank, the column add and the two stores
#pragma unroll 1
    for (int m0 = 0; m0 < G::ROWS; m0 += B) {
      T vb[B];
#pragma unroll
      for (int u = 0; u < B; u++) vb[u] = src[warp * G::PER_WARP + 32 * (m0 + u) + lane];
#pragma unroll
      for (int u = 0; u < B; u++) {
        const uint32_t e0 = warp * G::PER_WARP + 32 * (m0 + u);
        const uint32_t x0 = cbase + e0;
        const T v = vb[u];
        const uint32_t b = __ballot_sync(0xffffffffu, v != 0);
        const uint32_t r = lpre + __popc(b & lt);
        if (v != 0) {
          tcol[r] = (x0 & (C - 1)) + lane;
          tval[r] = v;
        }
        lpre += __popc(b);
        if (lane == 31 && (((x0 + 32) & (C - 1)) == 0 || p.tin + e0 + 32 == Fk))
          row_ptr[row0 + (x0 >> csh) + 1] = uint32_t(tile_off + lpre);
      }
    }
  } else {
#pragma unroll 1
    for (int m0 = 0; m0 < G::ROWS; m0 += B) {
      T vb[B];
#pragma unroll
      for (int u = 0; u < B; u++) {
        const uint32_t e = warp * G::PER_WARP + 32 * (m0 + u) + lane;
        vb[u] = (full || e < p.te) ? src[e] : T(0);
      }
#pragma unroll
      for (int u = 0; u < B; u++) {
        const uint32_t e = warp * G::PER_WARP + 32 * (m0 + u) + lane;
        const T v = vb[u];
        const uint32_t b = __ballot_sync(0xffffffffu, v != 0);
        const uint32_t r = lpre + __popc(b & lt);
        const uint32_t x = cbase + e;
        const uint32_t ro = pow2 ? x >> csh : x / C;
        const uint32_t col = x - ro * C;
        if (v != 0) {
          tcol[r] = col;
          tval[r] = v;
        }
        if ((full || e < p.te) && (col == C - 1 || p.tin + e + 1 == Fk))
          row_ptr[row0 + ro + 1] = uint32_t(tile_off + r + (v != 0));
        lpre += __popc(b);
      }
    }
  }
  if (tid == 0 && p.j == 0) row_ptr[0] = 0;
  if (tid == kThreads - 1 && p.tin + p.te == Fk) {  // last tile of the frame: section pads
    for (uint64_t b = 4 * (R + 1); b < a16(4 * (R + 1)); b += 4) *reinterpret_cast<uint32_t*>(out + fstart + b) = 0;
    uint8_t* cb = out + fstart + a16(4 * (R + 1));
    for (uint64_t b = 4 * nnz_k; b < a16(4 * nnz_k); b += 4) *reinterpret_cast<uint32_t*>(cb + b) = 0;
    uint8_t* vb = cb + a16(4 * nnz_k);
    for (uint64_t b = G::W * nnz_k; b < a16(G::W * nnz_k); b += 2) *reinterpret_cast<uint16_t*>(vb + b) = 0;
  }
}

template <typename T>
static cudaError_t csr_compress_t(const void* in, uint64_t n, uint64_t F, uint32_t C, uint8_t* out, uint64_t* out_size,
                                  const Scratch& sc, int dtype, cudaStream_t st) {
  using G = TileGeom<T>;
  const uint32_t K = uint32_t(cdiv(n, F));
  const uint32_t tpf = uint32_t(cdiv(F, G::TILE));
  const uint32_t tiles = rle_tiles(n, sizeof(T), F);
  const T* x = static_cast<const T*>(in);
  timing_kernel_start(st);
  CUDA_TRY_LAUNCH(pdl_launch(csr_count_kernel<T>, dim3(tiles), dim3(kThreads), 0, st, x, n, F, tpf, sc));
  CUDA_TRY_LAUNCH(pdl_launch(csr_scan_kernel<T>, dim3(K), dim3(1024), 0, st, n, F, tpf, C, sc));
  cudaError_t e = launch_finalize(out, kCSR, dtype, n, F, C, sc, out_size, st);
  if (e != cudaSuccess) return e;
  CUDA_TRY_LAUNCH(pdl_launch(csr_emit_kernel<T>, dim3(tiles), dim3(kThreads), 0, st, x, n, F, tpf, C, out, sc));
  return cudaGetLastError();
}

cudaError_t launch_csr_compress(const void* in, uint64_t n, int w, uint64_t F, uint32_t C, uint8_t* out,
                                uint64_t* out_size, const Scratch& sc, uint32_t /*epoch*/, int dtype, cudaStream_t st) {
  return w == 4 ? csr_compress_t<uint32_t>(in, n, F, C, out, out_size, sc, dtype, st)
                : csr_compress_t<uint16_t>(in, n, F, C, out, out_size, sc, dtype, st);
}

// ------------------------------------------------------------------------------------------
// decompress
// ------------------------------------------------------------------------------------------
#ifndef CSWAP_CSR_UNROLL
#define CSWAP_CSR_UNROLL 4
#endif
template <typename T>
__global__ void __launch_bounds__(kThreads) csr_expand_kernel(const uint8_t* __restrict__ in, T* __restrict__ outp,
                                                              uint64_t n, uint64_t F, uint32_t tpf, uint32_t C,
                                                              uint32_t k0, Scratch sc, uint32_t* err) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  using G = TileGeom<T>;
  __shared__ __align__(16) T s_x[G::TILE];
  __shared__ int s_bad;
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t t = blockIdx.x + k0 * tpf;
  const TilePos p = tile_pos<T>(t, n, F, tpf);
  const uint64_t R = cdiv(p.Fk, C);
  const uint64_t fstart = sc.aux[p.k], fb = sc.aux2[p.k];
  const uint32_t* row_ptr = reinterpret_cast<const uint32_t*>(in + fstart);
  if (tid == 0) s_bad = 0;
  for (uint32_t e = tid; e < G::TILE; e += kThreads) s_x[e] = 0;
  // frame-level consistency (every tile checks the sizes it relies on)
  uint64_t nnz = 0;
  bool ok = a16(4 * (R + 1)) <= fb;
  if (ok) {
    nnz = row_ptr[R];
    ok = row_ptr[0] == 0 && nnz <= p.Fk && fb == a16(4 * (R + 1)) + a16(4 * nnz) + a16(uint64_t(G::W) * nnz);
  }
  __syncthreads();
  if (ok) {
    const uint32_t* col = reinterpret_cast<const uint32_t*>(in + fstart + a16(4 * (R + 1)));
    const T* val = reinterpret_cast<const T*>(in + fstart + a16(4 * (R + 1)) + a16(4 * nnz));
    const uint64_t ra = p.tin / C, rb = (p.tin + p.te - 1) / C;
    bool bad = false;
    for (uint64_t r = ra + warp; r <= rb; r += kWarps) {  // one warp per row
      const uint64_t a = row_ptr[r], b = row_ptr[r + 1];
      const uint64_t width = (r + 1) * C <= p.Fk ? C : p.Fk - r * C;
      if (b < a || b > nnz) {
        bad = true;
        continue;
      }
      // column window of this tile inside row r
      const uint64_t rs = r * C;
      const uint64_t c_lo = p.tin > rs ? p.tin - rs : 0;
      const uint64_t c_hi = umin64(width, p.tin + p.te - rs);
      uint64_t q0 = a, q1 = b;
      if (c_lo > 0 || c_hi < width) {  // rows longer than the tile: binary-search the window
        uint64_t lo = a, hi = b;
        while (lo < hi) {
          const uint64_t mid = (lo + hi) / 2;
          if (col[mid] < c_lo) lo = mid + 1;
          else hi = mid;
        }
        q0 = lo;
        hi = b;
        while (lo < hi) {
          const uint64_t mid = (lo + hi) / 2;
          if (col[mid] < c_hi) lo = mid + 1;
          else hi = mid;
        }
        q1 = lo;
      }
      // U x 32 (col, value) pairs per step, all loads issued before the first use (the loop
      // was one dependent DRAM round trip per 32 pairs); the ascending-column check takes the
      // predecessor from the neighbouring lane, and from memory only for the window's first pair
      constexpr int U = CSWAP_CSR_UNROLL;
      uint32_t prev = (q0 > a && q0 < q1) ? col[q0 - 1] : 0u;  // column before the window
      bool has_prev = q0 > a;
      for (uint64_t qb = q0; qb < q1; qb += 32 * U) {
        uint32_t cv[U];
        T vv[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
          const uint64_t q = qb + uint64_t(u) * 32 + lane;
          cv[u] = q < q1 ? col[q] : 0u;
          vv[u] = q < q1 ? val[q] : T(0);
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
          const uint64_t q = qb + uint64_t(u) * 32 + lane;
          const uint32_t up = __shfl_up_sync(0xffffffffu, cv[u], 1);
          const uint32_t last = __shfl_sync(0xffffffffu, cv[u], 31);
          const uint32_t pc = lane ? up : prev;
          const bool hp = lane ? true : has_prev;
          if (q < q1) {
            const uint32_t c = cv[u];
            if (c >= width || (hp && pc >= c)) bad = true;
            else if (c >= c_lo && c < c_hi) s_x[rs + c - p.tin] = vv[u];
          }
          prev = last;
          has_prev = true;
        }
      }
    }
    if (bad) s_bad = 1;
  } else if (tid == 0) {
    s_bad = 1;
  }
  __syncthreads();
  if (s_bad) {
    if (tid == 0) set_error(err, kErrCorrupt);
    return;
  }
  T* dst = outp + uint64_t(p.k) * F + p.tin;
  constexpr int EPV = 16 / sizeof(T);
  const uint32_t nv = p.te / EPV;
  for (uint32_t v = tid; v < nv; v += kThreads)
    stg_stream(reinterpret_cast<uint4*>(dst) + v, reinterpret_cast<const uint4*>(s_x)[v]);
  for (uint32_t e = nv * EPV + tid; e < p.te; e += kThreads) dst[e] = s_x[e];
}

cudaError_t launch_csr_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t C,
                                  uint32_t k0, uint32_t k1, const Scratch& sc, uint32_t* err, cudaStream_t st) {
  if (k1 <= k0) return cudaSuccess;
  const uint32_t TILE = kTileBytes / w;
  const uint32_t tpf = uint32_t(cdiv(F, TILE));
  const uint32_t tiles = (k1 - 1 - k0) * tpf + uint32_t(cdiv(frame_len(n, F, k1 - 1), TILE));
  timing_kernel_start(st);
  if (w == 4)
    CUDA_TRY_LAUNCH(pdl_launch(csr_expand_kernel<uint32_t>, dim3(tiles), dim3(kThreads), 0, st, in, static_cast<uint32_t*>(out), n, F, tpf, C, k0, sc, err));
  else
    CUDA_TRY_LAUNCH(pdl_launch(csr_expand_kernel<uint16_t>, dim3(tiles), dim3(kThreads), 0, st, in, static_cast<uint16_t*>(out), n, F, tpf, C, k0, sc, err));
  return cudaGetLastError();
}

}  // namespace cswap
