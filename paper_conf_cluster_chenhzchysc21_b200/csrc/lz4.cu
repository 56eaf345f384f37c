// lz4.cu — LZ4 block codec for sm_100a.
//
// PAPER.md:220-222 (§IV-E): "LZ4 uses a dictionary-matching stage to reduce data size. For
// example, a string (abcde_bcde) can be compressed as (abcde_(5,4)), where 5 denotes the position
// how far back the redundant string (bcde) can be found and 4 denotes the length of matched
// string."  [25] = nvcomp: independent blocks.  Reading R6 / DESIGN.md §3.2: every
// B-byte block is an LZ4 *block-format* stream produced by the canonical greedy parse
// (MINMATCH 4, MFLIMIT 12, LASTLITERALS 5, HASHLOG 12, lookup-then-insert at every scanned
// position, nothing inserted inside matches).  Frame: u32 csize[nblk] pad16 | blocks | pad16.
//
// Compress: one warp per block (4 per CTA), the 4096-entry u16 hash table in shared memory, the
// block read through L1/L2.  The warp scans 32 consecutive positions at a time: lane j's
// candidate is the latest earlier lane with the same hash (__match_any_sync) else the table
// entry; the first lane whose candidate verifies ends the batch; lanes up to it insert (latest
// lane per hash wins).  This is exactly the sequential parse.  Matches are
// extended 32 bytes per step; sequences are written by the whole warp into a per-block scratch
// slot.  Then: per-frame scan of block sizes -> frame table -> pack (one CTA per block).
// Decompress: per-frame scan of csize -> block offsets; one warp per block decodes straight into
// the output (literal and match copies 32 bytes per step, short-offset matches by shuffling the
// `offset`-byte pattern) with every read and write bounds-checked.
#include "kernels.h"
#include "tile_common.cuh"

namespace cswap {

constexpr uint32_t kLz4MaxBlock = 65536;
constexpr uint32_t kLz4SlotBytes = 65824;  // >= L + L/255 + 16 for L = 65536, multiple of 16
constexpr uint16_t kLz4Empty = 0xFFFF;     // positions <= L-12 < 0xFFFF are the only ones inserted

__device__ __forceinline__ uint32_t le32_smem(const uint8_t* s, uint32_t p) {  // s 4-aligned, +8 pad
  const uint32_t* w = reinterpret_cast<const uint32_t*>(s);
  const uint32_t a = w[p >> 2], b = w[(p >> 2) + 1];
  return __funnelshift_r(a, b, (p & 3) * 8);
}

// Writes `len` bytes of `val` at out[op..] with the whole warp.
__device__ __forceinline__ void warp_fill(uint8_t* out, uint32_t op, uint32_t len, uint8_t val, int lane) {
  for (uint32_t q = lane; q < len; q += 32) out[op + q] = val;
}

// LZ4 length continuation for v >= 0 (the part beyond the token nibble): bytes of 255 + remainder
__device__ __forceinline__ uint32_t put_len_ext(uint8_t* out, uint32_t op, uint32_t v, int lane) {
  const uint32_t n255 = v / 255;
  warp_fill(out, op, n255, 255, lane);
  if (lane == 0) out[op + n255] = uint8_t(v - 255 * n255);
  return op + n255 + 1;
}

// Emit one sequence (literals src[anchor, anchor+nlit), optional match) at out[op]; returns new op.
__device__ __forceinline__ uint32_t emit_seq(uint8_t* out, uint32_t op, const uint8_t* src, uint32_t anchor,
                                             uint32_t nlit, bool has_match, uint32_t offset, uint32_t mlen, int lane) {
  const uint32_t tl = nlit < 15 ? nlit : 15;
  const uint32_t tm = has_match ? ((mlen - 4) < 15 ? (mlen - 4) : 15) : 0;
  if (lane == 0) out[op] = uint8_t((tl << 4) | tm);
  op++;
  if (nlit >= 15) op = put_len_ext(out, op, nlit - 15, lane);
  for (uint32_t q = lane; q < nlit; q += 32) out[op + q] = src[anchor + q];
  op += nlit;
  if (has_match) {
    if (lane == 0) {
      out[op] = uint8_t(offset & 0xFF);
      out[op + 1] = uint8_t(offset >> 8);
    }
    op += 2;
    if (mlen - 4 >= 15) op = put_len_ext(out, op, mlen - 4 - 15, lane);
  }
  return op;
}

// one warp per block; blocks indexed globally (frame-major), block b of frame k covers bytes
// [b*B, min((b+1)*B, Fk*w)) of the frame
// The source block is read through L1/L2 (it is not staged): only the 8 KiB hash table lives in
// shared memory, so 4 blocks per CTA and ~28 parsing warps per SM hide each other's latency
// (staging the 64 KiB block limited an SM to 3 warps: 7.6 GB/s at s = 0.5).
constexpr int kLz4Warps = 4;
constexpr uint32_t kLz4Ring = 4096;  // decode: recent-output ring per warp (power of two, >= 32)

__device__ __forceinline__ uint32_t le32_g(const uint8_t* s, uint32_t p) {  // s 16-aligned; p+8 <= block end
  const uint32_t* w = reinterpret_cast<const uint32_t*>(s);
  const uint32_t a = __ldg(w + (p >> 2)), b = __ldg(w + (p >> 2) + 1);
  return __funnelshift_r(a, b, (p & 3) * 8);
}

__global__ void __launch_bounds__(32 * kLz4Warps) lz4_compress_kernel(const uint8_t* __restrict__ in, uint64_t n,
                                                                      int w, uint64_t F, uint32_t B, uint32_t bpf,
                                                                      uint32_t nblk, uint8_t* slots, uint64_t* csize) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  __shared__ uint16_t s_tabs[kLz4Warps][4096];
  const int lane = threadIdx.x & 31;
  const uint32_t blk = blockIdx.x * kLz4Warps + (threadIdx.x >> 5);
  if (blk >= nblk) return;
  uint16_t* s_tab = s_tabs[threadIdx.x >> 5];
  const uint32_t k = blk / bpf, b = blk % bpf;
  const uint64_t fbytes = frame_len(n, F, k) * uint64_t(w);
  const uint32_t L = uint32_t(umin64(B, fbytes - uint64_t(b) * B));
  const uint8_t* s_src = in + uint64_t(k) * F * w + uint64_t(b) * B;  // global, read-only
  for (uint32_t h = lane; h < 4096; h += 32) s_tab[h] = kLz4Empty;
  __syncwarp();
  uint8_t* out = slots + uint64_t(blk) * kLz4SlotBytes;
  const uint32_t lt = (1u << lane) - 1u;
  uint32_t anchor = 0, i = 0, op = 0;
  if (L >= 13) {
    const uint32_t limit = L - 12;  // last position that may start a match
    while (i <= limit) {
      const uint32_t pos = i + lane;
      const bool active = pos <= limit;
      const uint32_t v = active ? le32_g(s_src, pos) : 0;
      const uint32_t h = active ? (v * 2654435761u) >> 20 : 0x10000u + lane;
      const uint32_t same = __match_any_sync(0xffffffffu, h);
      const uint32_t earlier = same & lt;
      uint32_t cand = kLz4Empty;
      if (active) cand = earlier ? i + (31 - __clz(earlier)) : s_tab[h];
      const bool ok = active && cand != kLz4Empty && le32_g(s_src, cand) == v;
      const uint32_t mm = __ballot_sync(0xffffffffu, ok);
      // lanes that insert: up to the first matching lane (all active lanes if none matched);
      // within a hash group the latest inserting lane wins
      const int f = mm ? __ffs(mm) - 1 : 31;
      const uint32_t upto = f == 31 ? 0xffffffffu : ((2u << f) - 1u);
      const uint32_t later = same & ~lt & ~(1u << lane) & upto;
      __syncwarp();
      if (active && (upto >> lane & 1u) && later == 0) s_tab[h] = uint16_t(pos);
      __syncwarp();
      if (!mm) {
        i += 32;
        continue;
      }
      const uint32_t mpos = i + f;
      const uint32_t c = __shfl_sync(0xffffffffu, cand, f);
      uint32_t len = 4;
      while (true) {  // extend while mpos+len < L-5 and bytes agree, 32 bytes per step
        const uint32_t q = mpos + len + lane;
        const bool eq = q < L - 5 && s_src[c + len + lane] == s_src[q];
        const uint32_t ne = __ballot_sync(0xffffffffu, !eq);
        if (ne) {
          len += __ffs(ne) - 1;
          break;
        }
        len += 32;
      }
      op = emit_seq(out, op, s_src, anchor, mpos - anchor, true, mpos - c, len, lane);
      i = mpos + len;
      anchor = i;
    }
  }
  op = emit_seq(out, op, s_src, anchor, L - anchor, false, 0, 0, lane);
  if (lane == 0) csize[blk] = op;
}

// one CTA per frame: block offsets inside the frame's block section (tbuf), frame_bytes (aux2)
__global__ void __launch_bounds__(1024) lz4_scan_kernel(uint64_t n, int w, uint64_t F, uint32_t B, uint32_t bpf,
                                                        Scratch sc) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  __shared__ uint64_t s_tmp[33];
  const uint32_t k = blockIdx.x;
  const uint32_t nb = uint32_t(cdiv(frame_len(n, F, k) * uint64_t(w), B));
  uint64_t* cs = sc.tbuf + uint64_t(k) * bpf;
  uint64_t* off = sc.tbuf2 + uint64_t(k) * bpf;
  uint64_t carry = 0;
  for (uint32_t c0 = 0; c0 < nb; c0 += blockDim.x) {
    const uint32_t j = c0 + threadIdx.x;
    const uint64_t v = j < nb ? cs[j] : 0;
    uint64_t tot;
    const uint64_t ex = block_excl_sum_u64(v, s_tmp, &tot);
    if (j < nb) off[j] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) sc.aux2[k] = a16(4ull * nb) + a16(carry);
}

// one CTA per block: copy the slot to its place, write csize[b], pads
__global__ void __launch_bounds__(256) lz4_pack_kernel(uint64_t n, int w, uint64_t F, uint32_t B, uint32_t bpf,
                                                       const uint8_t* slots, uint8_t* out, Scratch sc) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  const uint32_t blk = blockIdx.x;
  const uint32_t k = blk / bpf, b = blk % bpf;
  const uint32_t nb = uint32_t(cdiv(frame_len(n, F, k) * uint64_t(w), B));
  const uint64_t fstart = sc.aux[k];
  const uint64_t cs = sc.tbuf[blk];
  uint8_t* dst = out + fstart + a16(4ull * nb) + sc.tbuf2[blk];
  const uint8_t* src = slots + uint64_t(blk) * kLz4SlotBytes;
  for (uint32_t q = threadIdx.x; q < cs; q += blockDim.x) dst[q] = src[q];
  if (threadIdx.x == 0) reinterpret_cast<uint32_t*>(out + fstart)[b] = uint32_t(cs);
  if (threadIdx.x == 1 && b == nb - 1) {  // pads of the csize section and of the block section
    for (uint64_t q = 4ull * nb; q < a16(4ull * nb); q++) out[fstart + q] = 0;
    const uint64_t end = a16(4ull * nb) + sc.tbuf2[blk] + cs;
    for (uint64_t q = end; q < a16(end); q++) out[fstart + q] = 0;
  }
}

uint64_t lz4_scratch_bytes(uint64_t n, int w, uint64_t F, uint32_t B) {
  const uint64_t K = cdiv(n, F);
  uint64_t nblk = 0;
  for (uint64_t k = 0; k < K; k++) nblk += cdiv(frame_len(n, F, k) * w, B);
  return (nblk + 1) * kLz4SlotBytes;
}

static uint32_t lz4_blocks(uint64_t n, int w, uint64_t F, uint32_t B, uint32_t* bpf_out) {
  const uint32_t K = uint32_t(cdiv(n, F));
  const uint32_t bpf = uint32_t(cdiv(F * w, B));
  if (bpf_out) *bpf_out = bpf;
  return (K - 1) * bpf + uint32_t(cdiv(frame_len(n, F, K - 1) * w, B));
}

cudaError_t launch_lz4_compress(const void* in, uint64_t n, int w, uint64_t F, uint32_t B, uint8_t* out,
                                uint64_t* out_size, uint8_t* slots, const Scratch& sc, int dtype, cudaStream_t st) {
  const uint32_t K = uint32_t(cdiv(n, F));
  uint32_t bpf;
  const uint32_t nblk = lz4_blocks(n, w, F, B, &bpf);
  timing_kernel_start(st);
  CUDA_TRY_LAUNCH(pdl_launch(lz4_compress_kernel, dim3((nblk + kLz4Warps - 1) / kLz4Warps), dim3(32 * kLz4Warps), 0, st, 
      static_cast<const uint8_t*>(in), n, w, F, B, bpf, nblk, slots, sc.tbuf));
  CUDA_TRY_LAUNCH(pdl_launch(lz4_scan_kernel, dim3(K), dim3(1024), 0, st, n, w, F, B, bpf, sc));
  cudaError_t e = launch_finalize(out, kLZ4, dtype, n, F, B, sc, out_size, st);
  if (e != cudaSuccess) return e;
  CUDA_TRY_LAUNCH(pdl_launch(lz4_pack_kernel, dim3(nblk), dim3(256), 0, st, n, w, F, B, bpf, slots, out, sc));
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// decompress
// ------------------------------------------------------------------------------------------
// one CTA per frame: validate csize against frame_bytes, block offsets -> tbuf2
__global__ void __launch_bounds__(1024) lz4_dscan_kernel(const uint8_t* __restrict__ in, uint64_t n, int w,
                                                         uint64_t F, uint32_t B, uint32_t bpf, uint32_t k0, Scratch sc,
                                                         uint32_t* err) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  __shared__ uint64_t s_tmp[33];
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const uint32_t k = k0 + blockIdx.x;
  const uint32_t nb = uint32_t(cdiv(frame_len(n, F, k) * uint64_t(w), B));
  const uint64_t fstart = sc.aux[k], fb = sc.aux2[k];
  if (a16(4ull * nb) > fb) {
    if (threadIdx.x == 0) set_error(err, kErrCorrupt);
    return;
  }
  const uint32_t* cs = reinterpret_cast<const uint32_t*>(in + fstart);
  uint64_t* off = sc.tbuf2 + uint64_t(k) * bpf;
  uint64_t* csz = sc.tbuf + uint64_t(k) * bpf;
  uint64_t carry = 0;
  for (uint32_t c0 = 0; c0 < nb; c0 += blockDim.x) {
    const uint32_t j = c0 + threadIdx.x;
    const uint64_t v = j < nb ? cs[j] : 0;
    uint64_t tot;
    const uint64_t ex = block_excl_sum_u64(v, s_tmp, &tot);
    if (j < nb) {
      off[j] = carry + ex;
      csz[j] = v;
    }
    carry += tot;
  }
  if (threadIdx.x == 0 && a16(4ull * nb) + a16(carry) != fb) set_error(err, kErrCorrupt);
}

// One warp per block, writing straight into the output tensor (no shared-memory staging, so
// ~16 warps per SM); match sources are read back with ld.global.cg (L2, coherent with the
// warp's own earlier stores after __syncwarp).
__device__ __forceinline__ uint8_t ld_cg_u8(const uint8_t* p) {
  uint16_t v;
  asm volatile("ld.global.cg.u8 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
  return uint8_t(v);
}

__global__ void __launch_bounds__(32 * kLz4Warps) lz4_decode_kernel(const uint8_t* __restrict__ in, uint8_t* outp,
                                                                    uint64_t n, int w, uint64_t F, uint32_t B,
                                                                    uint32_t bpf, uint32_t k0, uint32_t nslots,
                                                                    Scratch sc, uint32_t* err) {
  pdl_trigger();  // PDL: the next kernel of the group may launch now
  pdl_wait();     // ... and this one reads its predecessor's output only after it completed
  // the warp's last kLz4Ring output bytes (ring indexed by output position): match sources within
  // that distance are read from shared memory, not back from L2 (an L2 round trip per match
  // bounded the decode at ~55 GB/s for ReLU data, whose matches are mostly a few bytes back)
  __shared__ __align__(16) uint8_t s_rings[kLz4Warps][kLz4Ring];
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const int lane = threadIdx.x & 31;
  const uint32_t slot = blockIdx.x * kLz4Warps + (threadIdx.x >> 5);
  if (slot >= nslots) return;
  uint8_t* ring = s_rings[threadIdx.x >> 5];
  constexpr uint32_t RM = kLz4Ring - 1;
  const uint32_t k = k0 + slot / bpf, b = slot % bpf;
  const uint64_t fbytes = frame_len(n, F, k) * uint64_t(w);
  const uint32_t nb = uint32_t(cdiv(fbytes, B));
  if (b >= nb) return;
  const uint32_t L = uint32_t(umin64(B, fbytes - uint64_t(b) * B));
  const uint64_t blk = uint64_t(k) * bpf + b;
  const uint64_t fstart = sc.aux[k], fb = sc.aux2[k];
  const uint64_t cs64 = sc.tbuf[blk];
  const uint64_t start = a16(4ull * nb) + sc.tbuf2[blk];
  // a valid block is at most LZ4's bound for L bytes, so the parse runs on 32-bit offsets
  bool bad = start + cs64 > fb || cs64 > uint64_t(L) + L / 255 + 16;
  const uint32_t cs = bad ? 0u : uint32_t(cs64);
  const uint8_t* ip0 = in + fstart + start;
  uint8_t* dst = outp + uint64_t(k) * F * w + uint64_t(b) * B;
  uint32_t ip = 0;
  uint32_t op = 0;
  auto rd = [&](uint32_t at) -> uint32_t { return at < cs ? __ldg(ip0 + at) : 0u; };
  while (!bad) {
    if (ip >= cs) { bad = true; break; }
    const uint32_t token = rd(ip++);
    uint32_t nlit = token >> 4;
    if (nlit == 15) {
      uint32_t x;
      do {
        if (ip >= cs) { bad = true; break; }
        x = rd(ip++);
        nlit += x;
      } while (x == 255);
      if (bad) break;
    }
    if (ip + nlit > cs || op + nlit > L) { bad = true; break; }
    for (uint32_t q = lane; q < nlit; q += 32) {
      const uint8_t x = __ldg(ip0 + ip + q);
      dst[op + q] = x;
      ring[(op + q) & RM] = x;
    }
    ip += nlit;
    op += nlit;
    if (ip == cs) break;  // last sequence: literals only
    if (ip + 2 > cs) { bad = true; break; }
    const uint32_t offset = rd(ip) | (rd(ip + 1) << 8);
    ip += 2;
    uint32_t mlen = token & 15;
    if (mlen == 15) {
      uint32_t x;
      do {
        if (ip >= cs) { bad = true; break; }
        x = rd(ip++);
        mlen += x;
      } while (x == 255);
      if (bad) break;
    }
    mlen += 4;
    if (offset == 0 || offset > op || op + mlen > L) { bad = true; break; }
    __syncwarp();  // the match source may have been written by other lanes
    if (offset >= 32) {  // non-overlapping within a 32-byte step
      // source still in the ring, and not in a slot this 32-byte step overwrites (a step writes
      // positions up to o + 31, i.e. ring slots of positions up to 31 bytes past o - kLz4Ring;
      // compute-sanitizer racecheck found offsets 4065..4095 racing before this bound)
      const bool near = offset + 32 <= kLz4Ring;
      for (uint32_t q = 0; q < mlen; q += 32) {
        if (q + lane < mlen) {
          const uint32_t o = op + q + lane;
          const uint8_t x = near ? ring[(o - offset) & RM] : ld_cg_u8(dst + o - offset);
          dst[o] = x;
          ring[o & RM] = x;
        }
        __syncwarp();
      }
    } else {  // short offset: the match repeats the last `offset` bytes
      const uint32_t base = op - offset;
      const uint32_t pat = lane < int(offset) ? ring[(base + lane) & RM] : 0u;
      for (uint32_t q0 = 0; q0 < mlen; q0 += 32) {  // whole-warp iterations: every lane shuffles
        const uint32_t q = q0 + lane;
        const uint32_t v = __shfl_sync(0xffffffffu, pat, q % offset);
        if (q < mlen) {
          dst[op + q] = uint8_t(v);
          ring[(op + q) & RM] = uint8_t(v);
        }
      }
    }
    op += mlen;
    __syncwarp();
  }
  if (!bad && op != L) bad = true;
  if (__any_sync(0xffffffffu, bad) && lane == 0) set_error(err, kErrCorrupt);
}

cudaError_t launch_lz4_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t B,
                                  uint32_t k0, uint32_t k1, const Scratch& sc, uint32_t* err, cudaStream_t st) {
  if (k1 <= k0) return cudaSuccess;
  const uint32_t bpf = uint32_t(cdiv(F * w, B));
  timing_kernel_start(st);
  CUDA_TRY_LAUNCH(pdl_launch(lz4_dscan_kernel, dim3(k1 - k0), dim3(1024), 0, st, in, n, w, F, B, bpf, k0, sc, err));
  const uint32_t nslots = (k1 - k0) * bpf;
  CUDA_TRY_LAUNCH(pdl_launch(lz4_decode_kernel, dim3((nslots + kLz4Warps - 1) / kLz4Warps), dim3(32 * kLz4Warps), 0, st, 
      in, static_cast<uint8_t*>(out), n, w, F, B, bpf, k0, nslots, sc, err));
  return cudaGetLastError();
}

}  // namespace cswap
