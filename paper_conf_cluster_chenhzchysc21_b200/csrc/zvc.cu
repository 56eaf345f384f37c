// zvc.cu — zero-value compression (ZVC) for sm_100a.
//
// PAPER.md:222 (§IV-E): "Similar to CSR, ZVC stores a float sequence as non-zero values and
// additional indexes ... it utilizes a 32-bit bitmap as the index for 32 consecutive floats".
// Byte layout: DESIGN.md §3 (frame = u32 bitmap[ceil(Fk/32)] pad16 | non-zero words pad16).
//
// Compress (one pass over the input): a persistent, warp-specialised kernel.
//   producer warp: streams the CTA's tiles (static round robin) into a ring of shared-memory
//           stages with cp.async.bulk (TMA 1-D) + mbarrier completion;
//   consumer warps: count tile i (warp ballots -> bitmap words, per-lane ranks, in-place
//           compaction) and publish its count, then emit tile i-LAG at its container offset;
//   resolver warps (one per stage): the tile's absolute offset from the published COUNTS of the
//           earlier tiles of its frame (per-frame and 32-tile-group accumulators), no chained
//           prefixes.
// Decompress (no inter-CTA waiting): tile popcounts of the bitmap (reads n/8 B),
// a per-frame scan of those counts into value offsets, then one CTA per tile pulls its bitmap
// slice and value span into shared memory with cp.async.bulk and expands with 128-bit stores.
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <atomic>
#include <type_traits>

#include "common.cuh"
#include "kernels.h"

namespace cswap {

// optional phase profiling of the persistent compress kernel (CSWAP_ZVC_PROF=1)
__device__ unsigned long long g_zprof[16];
#define ZPROF_ADD(i, v) \
  do {                  \
    if (prof) atomicAdd(&g_zprof[i], (unsigned long long)(v)); \
  } while (0)

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

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(bar)))
               : "memory");
}

// ------------------------------------------------------------------------------------------
// compress: persistent, warp-specialised
//   warp 8  producer: ticket + cp.async.bulk of the tile into stage s          (bar_full[s])
//   warp 9  resolver: container offset of the tile's values = frame start + bitmap + W x
//                     (totals of the earlier 32-tile groups of the frame + counts of the
//                     earlier tiles of its group), all read from published COUNTS  (bar_off[s])
//   warps 0-7 consumers, per tile: (a) rows of 32 elements -> one ballot = one bitmap word,
//                     ranks from popcounts (no shuffles); publish the tile count and add it to
//                     the frame / group accumulators                           (bar_cnt[s]);
//                     (b) in-place compaction inside the stage (needs no offset); later
//                     (c) wait for the offset, copy the packed bytes out with 128-bit stores at
//                     the destination's 16-byte phase, store the bitmap slice, release the
//                     stage                                                    (bar_empty[s])
//   The consumers run (a)(b) of tile i+1 before (c) of tile i, so the offset latency overlaps.
// ------------------------------------------------------------------------------------------
// warps [0, CW) consumers, warp CW producer, warps CW+1 .. CW+S resolvers: one resolver warp per
// stage, so a resolver only ever waits on its own stage's barriers and can never observe another
// phase's parity
template <int S, int CW>
constexpr int compress_threads() { return 32 * (CW + 1 + S); }

// resolver polling: __nanosleep backoff bounds (ns).  A/B x2 of 32 / 16 / 8 ns / no sleep
// (profiles/zvc_backoff_ab_r02.jsonl): 8 ns is fastest or tied everywhere (1 GiB f32 s = 0.5
// 0.332 -> 0.326 ms, s = 0.8 0.303 -> 0.297; 256 MiB -2 %; f16 -0.5..1 %): a resolver that
// learns a count sooner releases the consumers' emit sooner; spinning without a sleep takes
// issue slots from the consumers (worse than 8 ns)
#ifndef CSWAP_ZVC_MAX_BACKOFF
#define CSWAP_ZVC_MAX_BACKOFF 8
#endif
#ifndef CSWAP_ZVC_MIN_BACKOFF
#define CSWAP_ZVC_MIN_BACKOFF 8
#endif
constexpr uint32_t kMinBackoff = CSWAP_ZVC_MIN_BACKOFF, kMaxBackoff = CSWAP_ZVC_MAX_BACKOFF;
// one resolver poll pause: __nanosleep with exponential backoff (kMaxBackoff = 0: spin)
__device__ __forceinline__ void resolver_pause(uint32_t& backoff) {
  if (kMaxBackoff == 0) return;
  __nanosleep(backoff);
  backoff = backoff < kMaxBackoff ? backoff * 2 : kMaxBackoff;
}
// accumulator words (per frame, per 32-tile group, per frame done-count, the CTA counter) are
// CSWAP_ZVC_ACC_STRIDE u64 apart: 16 puts each on its own 128-byte line.  Packed, a frame's 16
// group words shared one line that every consumer's atomics and every resolver's polls hit;
// A/B x2 (profiles/zvc_accstride_ab_r02.jsonl): 1 GiB f32 0.328 -> 0.322 ms (s = 0.5), 0.301 ->
// 0.293 (s = 0.8), 0.291 -> 0.283 (s = 0.95); 96 / 256 MiB f32 -2..4 %; 16-bit unchanged
#ifndef CSWAP_ZVC_ACC_STRIDE
#define CSWAP_ZVC_ACC_STRIDE 16
#endif
constexpr uint64_t kAccStride = CSWAP_ZVC_ACC_STRIDE;
// tile status words CSWAP_ZVC_STATUS_STRIDE u64 apart: each tile's count is stored once by its
// CTA and polled by the resolvers of the later tiles of its group; packed four to a 32-byte
// sector, neighbouring CTAs' stores and those polls met on the same sectors.  A/B x2
// (profiles/zvc_statusstride_ab_r02.jsonl): stride 2 and 16 equal, 1 GiB f32 0.320 -> 0.309 ms
// (s = 0.5), 0.281 -> 0.276 (s = 0.95), 96 / 256 MiB f32 -2..5 %, f16 -0.5..1 %
#ifndef CSWAP_ZVC_STATUS_STRIDE
#define CSWAP_ZVC_STATUS_STRIDE 2
#endif
constexpr uint64_t kStatusStride = CSWAP_ZVC_STATUS_STRIDE;
// 1: a per-frame accumulator (one atomic per tile) gives the next frame its start; 0: the next
// frame's first resolver sums the frame's 32-tile group accumulators instead (one hot word and
// one atomic per tile fewer; A/B x2, profiles/zvc_frameacc_ab_r02.jsonl: f16 1 GiB -1..1.5 %,
// f32 0..-0.7 %)
#ifndef CSWAP_ZVC_FRAMEACC
#define CSWAP_ZVC_FRAMEACC 0
#endif
// decode chain: each kernel triggers its dependent's launch as it starts (PDL)
#ifndef CSWAP_PDL_TRIGGER
#define CSWAP_PDL_TRIGGER 1
#endif
#ifndef CSWAP_ZVC_POW2
#define CSWAP_ZVC_POW2 1
#endif
#ifndef CSWAP_ZVC_PF
#define CSWAP_ZVC_PF 1
#endif
#ifndef CSWAP_ZVC_BM4
#define CSWAP_ZVC_BM4 1
#endif
// rows per batch of count_slab's loads
#ifndef CSWAP_ZVC_BATCH
#define CSWAP_ZVC_BATCH 4
#endif
// mbarrier waits sleep between tests (max ns): the producer refills a stage whose TMA load takes
// ~1 us anyway; a resolver has LAG tile periods (~1.5 us each) before its offset is needed; the
// polling consumer warp is on the critical path and sleeps least
#ifndef CSWAP_ZVC_SLEEP
#define CSWAP_ZVC_SLEEP 1
#endif
constexpr uint32_t kProducerSleep = 256 * CSWAP_ZVC_SLEEP, kResolverSleep = 128 * CSWAP_ZVC_SLEEP,
                   kConsumerSleep = 64 * CSWAP_ZVC_SLEEP;
// how the producer (bar_empty) and the consumers' polling warp (bar_full) wait: 0 = test +
// __nanosleep backoff, 1 = mbarrier.try_wait, which suspends the warp in hardware until the phase
// completes or ~4 us pass (tools/sleep_probe.cu: one instruction per wake-up instead of one poll
// per 66-513 ns of __nanosleep).  A/B at 1 GiB f32 / f16 and 96 MiB: the same times within the
// event timer's 2 us steps (the kernel is latency-bound in the consumers, not issue-bound), so
// 1 is kept for the issue slots it leaves to kernels sharing the SMs

#ifndef CSWAP_ZVC_PWAIT
#define CSWAP_ZVC_PWAIT 1
#endif
#ifndef CSWAP_ZVC_CWAIT
#define CSWAP_ZVC_CWAIT 1
#endif
__device__ __forceinline__ void producer_wait(uint64_t* bar, uint32_t parity) {
  if (CSWAP_ZVC_PWAIT) mbar_wait(bar, parity);
  else mbar_wait_sleep(bar, parity, kProducerSleep);
}

// the resolver handshakes (tile counted -> resolver; offset resolved -> consumers) on named
// barriers (bar.arrive / bar.sync: a waiting warp issues nothing) instead of polled mbarriers
// (ncu, f16 1 GiB: the polling loops were 39 % of all issued instructions)
#ifndef CSWAP_ZVC_NAMED
#define CSWAP_ZVC_NAMED 1
#endif
constexpr bool kNamedBars = CSWAP_ZVC_NAMED != 0;
__device__ __forceinline__ void named_arrive(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ void named_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

#ifndef CSWAP_ZVC_DYNAMIC_TILES
constexpr bool kStaticTiles = true;
#else
constexpr bool kStaticTiles = false;
#endif

// store of one 16- or 32-bit word at a shared byte address.  Only the in-place compaction uses
// it: its stores land at or before the rows already loaded (count_slab), so the compiler may move
// later loads across it (no "memory" clobber).
template <typename T>
__device__ __forceinline__ void sts_word(uint32_t a, uint32_t x) {
  if constexpr (sizeof(T) == 4) asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(x));
  else asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"(uint16_t(x)));
}

// a * W + c, opaque to the front end's reassociation (which would otherwise turn the running
// byte address back into an element count plus a scaled add per store)
template <int W>
__device__ __forceinline__ uint32_t mad_u32(uint32_t a, uint32_t c) {
  uint32_t r;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "n"(W), "r"(c));
  return r;
}

#ifndef CSWAP_ZVC_ROWASM
#define CSWAP_ZVC_ROWASM 1
#endif
// One row of the compacting count: p = (x != 0); w = ballot(p); @p store x at the shared byte
// address sdp + W * popc(w & lt); sdp += W * popc(w).  A single predicate register serves the
// ballot and the store.
template <typename T>
__device__ __forceinline__ void row_compact(uint32_t x, uint32_t lt, uint32_t& sdp, uint32_t& w) {
  if constexpr (sizeof(T) == 4) {
    asm("{\n\t.reg .pred p;\n\t.reg .b32 r, a;\n\t"
        "setp.ne.u32 p, %2, 0;\n\t"
        "vote.sync.ballot.b32 %0, p, 0xffffffff;\n\t"
        "and.b32 r, %0, %3;\n\t"
        "popc.b32 r, r;\n\t"
        "mad.lo.u32 a, r, 4, %1;\n\t"
        "@p st.shared.u32 [a], %2;\n\t"
        "popc.b32 r, %0;\n\t"
        "mad.lo.u32 %1, r, 4, %1;\n\t}"
        : "=&r"(w), "+r"(sdp)
        : "r"(x), "r"(lt)
        : "memory");
  } else {
    asm("{\n\t.reg .pred p;\n\t.reg .b32 r, a;\n\t.reg .b16 h;\n\t"
        "setp.ne.u32 p, %2, 0;\n\t"
        "vote.sync.ballot.b32 %0, p, 0xffffffff;\n\t"
        "and.b32 r, %0, %3;\n\t"
        "popc.b32 r, r;\n\t"
        "mad.lo.u32 a, r, 2, %1;\n\t"
        "cvt.u16.u32 h, %2;\n\t"
        "@p st.shared.u16 [a], h;\n\t"
        "popc.b32 r, %0;\n\t"
        "mad.lo.u32 %1, r, 2, %1;\n\t}"
        : "=&r"(w), "+r"(sdp)
        : "r"(x), "r"(lt)
        : "memory");
  }
}

// compress tile geometry: TB bytes per tile
template <typename T, int TB>
struct CGeom {
  static constexpr int W = sizeof(T);
  static constexpr int TILE = TB / W;  // elements per tile
  static constexpr int WT = TILE / 32;  // bitmap words per tile
};

template <typename T, int S, int TB>
struct CompressSmem {
  using G = CGeom<T, TB>;
  static constexpr uint32_t in_off = 0;
  static constexpr uint32_t bytes = S * TB + 128;  // dynamic: the stage ring (+ pad)
  static constexpr uint32_t static_bytes = S * G::WT * 4 + 1024;  // bitmap words, barriers, ...
  // resident CTAs per SM allowed by shared memory (228 KiB per SM, 1 KiB reserved per CTA), max 4
  static constexpr int by_smem = int((228u * 1024u) / (bytes + static_bytes + 1024u));
  static constexpr int ctas_per_sm = by_smem > 4 ? 4 : (by_smem < 1 ? 1 : by_smem);
};

// S stages; CW consumer warps; the consumers count tile i and emit tile i - LAG (LAG = S - 2),
// so a tile's offset has LAG count phases of slack to resolve.
template <typename T, int S, int CW, int TB>
__global__ void __launch_bounds__(compress_threads<S, CW>(), CompressSmem<T, S, TB>::ctas_per_sm)
    zvc_compress_persistent(const T* __restrict__ in, uint64_t n, uint64_t F, uint32_t K, uint32_t tpf,
                            uint32_t num_tiles, uint8_t* __restrict__ out, uint64_t* out_size, Scratch sc,
                            uint32_t epoch, int dtype, int prof) {
  const uint32_t gpf = (tpf + 31) / 32;  // 32-tile groups per frame
  using G = CGeom<T, TB>;
  using L = CompressSmem<T, S, TB>;
  constexpr uint32_t SENT = 0xFFFFFFFFu;
  constexpr int kProducerWarp = CW;
  constexpr int LAG = S - 2;
  // named barriers: 0 = __syncthreads, 1 = consumer_sync, then per stage count / offset
  constexpr uint32_t kBarCnt0 = 2, kBarOff0 = 2 + S;
  static_assert(kBarOff0 + S <= 16, "named barrier ids");
  constexpr int PW = G::TILE / CW;   // elements per consumer warp (slab) per tile
  constexpr int WPW = G::WT / CW;    // bitmap words per slab
  static_assert(LAG >= 1 && PW % 256 == 0, "compress geometry");
  extern __shared__ __align__(128) uint8_t smem[];
  uint8_t* s_in = smem + L::in_off;
  // [S][WT] bitmap words per stage: a separate (static) array, so the compiler knows the
  // bitmap stores never alias the stage loads and can batch the loads of a slab
  __shared__ __align__(16) uint32_t s_bm[S * G::WT];
  __shared__ __align__(8) uint64_t bar_full[S], bar_empty[S], bar_cnt[S], bar_off[S];
  __shared__ uint32_t s_ticket[S];
  __shared__ uint32_t s_nnz[S];
  __shared__ uint32_t s_wtot[S][CW];  // non-zeros per slab, per stage
  __shared__ uint64_t s_off[S], s_fs[S];

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    if (sc.kclock && blockIdx.x == 0) sc.kclock[0] = globaltimer_ns();  // the grid is co-resident (cooperative)
    for (int s = 0; s < S; s++) {
      mbar_init(&bar_full[s], 1);
      mbar_init(&bar_empty[s], CW);
      mbar_init(&bar_cnt[s], 1);
      mbar_init(&bar_off[s], 1);
    }
  }
  __syncthreads();

  const bool tpf_pow2 = CSWAP_ZVC_POW2 && (tpf & (tpf - 1)) == 0;
  const int tpf_sh = __ffs(int(tpf)) - 1;
  auto tile_geom = [&](uint32_t t, uint32_t& k, uint32_t& j, uint64_t& Fk, uint32_t& tile_elems,
                       uint32_t& bulk_elems) {
    k = tpf_pow2 ? t >> tpf_sh : t / tpf;  // tiles per frame is a power of two for power-of-two
    j = tpf_pow2 ? t & (tpf - 1) : t % tpf;  // frames: a shift instead of a ~20-instruction divide
    Fk = frame_len(n, F, k);
    tile_elems = uint32_t(umin64(G::TILE, Fk - uint64_t(j) * G::TILE));
    bulk_elems = ((tile_elems * G::W) & ~15u) / G::W;
  };

  if (warp == kProducerWarp) {  // ----------------------------------------- producer (TMA)
    // swap-out progress (sc.prog): once a stage's previous tile is fully emitted (bar_empty:
    // every consumer warp arrived after its stores, mbarrier arrive = release.cta, wait =
    // acquire.cta), count it for its frame with a gpu-scope acq_rel atomic; the CTA that
    // completes a frame publishes the frame's end offset (frame start + its frame-table entry,
    // both written before the frame's last tiles were emitted) for the host's per-frame D2H
    uint64_t* const fdone = sc.zacc + (K + uint64_t(K) * gpf) * kAccStride;  // after the accumulators
    auto tile_emitted = [&](uint32_t t) {
      if (!sc.prog || sc.prog_mode != 1 || lane != 0) return;
      uint32_t k, j, te, be;
      uint64_t Fk;
      tile_geom(t, k, j, Fk, te, be);
      unsigned long long old;
      asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], 1;"
                   : "=l"(old)
                   : "l"(fdone + k * kAccStride)
                   : "memory");
      if (old + 1 == cdiv(Fk, G::TILE)) {
        const uint64_t fs = status_value(ld_relaxed(sc.aux + k));
        const uint64_t fb = ld_relaxed(reinterpret_cast<const uint64_t*>(out + 64) + k);
        publish_frame(sc.prog, k, fs + fb);
      }
    };
    uint32_t i = 0;
    for (;; i++) {
      const int s = i % S;
      long long c0 = clock64();
      // the tile of round i - S (this stage's previous tile); counted for its frame only after
      // the stage is refilled, so the atomic's round trip never delays the next TMA load
      uint32_t done_t = SENT;
      if (i >= S) {
        producer_wait(&bar_empty[s], ((i / S) - 1) & 1);
        if (lane == 0) done_t = s_ticket[s];  // lane 0 alone reads and (below) rewrites the slot
      }
      if (lane == 0) ZPROF_ADD(0, clock64() - c0);
      // static round-robin assignment: CTA b takes tiles b, b + G, b + 2G, ... so every CTA
      // counts the tiles of round r at about the same time and a tile's offset waits only for
      // the skew between CTAs (a dynamic ticket would be claimed up to S-1 tiles before it is
      // counted, and later tiles would wait for that prefetch lag)
      const uint32_t t = kStaticTiles ? blockIdx.x + i * gridDim.x
                                      : __shfl_sync(0xffffffffu, lane == 0 ? atomicAdd(sc.tickets + epoch, 1u) : 0u, 0);
      if (t >= num_tiles) {
        if (lane == 0) {
          s_ticket[s] = SENT;
          mbar_arrive(&bar_full[s]);
        }
        if (done_t != SENT) tile_emitted(done_t);
        // the tiles of rounds i-S+1 .. i-1 are still being emitted: wait for each and count it
        if (sc.prog && sc.prog_mode == 1) {
          for (uint32_t p = i >= uint32_t(S - 1) ? i - (S - 1) : 0; p < i; p++) {
            producer_wait(&bar_empty[p % S], (p / S) & 1);
            if (lane == 0) tile_emitted(s_ticket[p % S]);
          }
        }
        break;
      }
      if (lane == 0) {
        uint32_t k, j, te, be;
        uint64_t Fk;
        tile_geom(t, k, j, Fk, te, be);
        s_ticket[s] = t;
        if (be) {
          mbar_expect_tx(&bar_full[s], be * G::W);
          bulk_g2s(s_in + s * TB, in + uint64_t(k) * F + uint64_t(j) * G::TILE, be * G::W, &bar_full[s]);
        } else {
          mbar_arrive(&bar_full[s]);
        }
      }
      if (done_t != SENT) tile_emitted(done_t);
    }
  } else if (warp > kProducerWarp) {  // ------------------------- resolvers (one per stage)
    const int r = warp - kProducerWarp - 1;
    for (uint32_t i = r;; i += S) {
      const int s = r;
      long long c0 = clock64();
      if (kNamedBars) named_sync(kBarCnt0 + s, 64);
      else mbar_wait_sleep(&bar_cnt[s], (i / S) & 1, kResolverSleep);
      long long c1 = clock64();
      if (lane == 0) ZPROF_ADD(2, c1 - c0);
      const uint32_t nnz = s_nnz[s];
      if (nnz == SENT) break;
      const uint32_t t = s_ticket[s];
      const uint32_t k = tpf_pow2 ? t >> tpf_sh : t / tpf, j = tpf_pow2 ? t & (tpf - 1) : t % tpf;
      const uint64_t nwords_k = cdiv(frame_len(n, F, k), 32);
      uint64_t excl = 0, fstart = 0;
      // offset = frame start + bitmap + W * (totals of earlier 32-tile groups of the frame +
      // counts of earlier tiles of the group).  Everything comes from COUNTS (published as soon
      // as a tile lands), never from other tiles' resolutions, so no chain forms across tiles.
      if (!CSWAP_ZVC_FRAMEACC && j == 0 && k > 0) {
        // previous frame's start + its bitmap + its packed values, the values summed from the
        // previous frame's group accumulators (lane l: groups l, l + 32, ...), each complete
        const uint64_t Fp = frame_len(n, F, k - 1);
        const uint32_t tiles_prev = uint32_t(cdiv(Fp, G::TILE)), gp = (tiles_prev + 31) / 32;
        uint64_t nz = 0;
        for (uint32_t gi = lane; gi < gp; gi += 32) {
          const uint64_t* p = sc.zacc + (K + uint64_t(k - 1) * gpf + gi) * kAccStride;
          const uint64_t want = gi + 1 < gp ? 32 : tiles_prev - 32 * gi;
          uint64_t v;
          uint32_t backoff = kMinBackoff;
          while (((v = ld_relaxed(p)) >> 40) != want) resolver_pause(backoff);
          nz += v & ((1ull << 40) - 1);
        }
        nz = warp_sum_u64(nz);
        if (lane == 0) {
          uint64_t a;
          uint32_t backoff = kMinBackoff;
          while (status_flag(a = ld_relaxed(sc.aux + k - 1), epoch) != kFlagP) resolver_pause(backoff);
          fstart = status_value(a) + a16(4 * cdiv(Fp, 32)) + a16(G::W * nz);
          st_relaxed(sc.aux + k, make_status(fstart, epoch, kFlagP));
        }
      } else if (j == 0 && lane == 0) {
        if (k == 0) {
          fstart = data_start(K);
        } else {  // previous frame's start + its bitmap + its packed values (from its accumulator)
          uint64_t a, acc;
          uint32_t backoff = kMinBackoff;
          while (status_flag(a = ld_relaxed(sc.aux + k - 1), epoch) != kFlagP) {
            resolver_pause(backoff);
          }
          const uint64_t Fp = frame_len(n, F, k - 1);
          const uint64_t tiles_prev = cdiv(Fp, G::TILE);
          backoff = kMinBackoff;
          while (((acc = ld_relaxed(sc.zacc + (k - 1) * kAccStride)) >> 40) != tiles_prev) {
            resolver_pause(backoff);
          }
          fstart = status_value(a) + a16(4 * cdiv(Fp, 32)) + a16(G::W * (acc & ((1ull << 40) - 1)));
        }
        st_relaxed(sc.aux + k, make_status(fstart, epoch, kFlagP));
      }
      uint64_t prefix = 0;  // non-zeros of the frame before this tile
      {
        const uint32_t g = j / 32;
        for (uint32_t g0 = 0; g0 < g; g0 += 32) {  // complete groups before g (32 tiles each)
          const uint32_t gi = g0 + lane;
          uint64_t v = 0;
          if (gi < g) {
            const uint64_t* p = sc.zacc + (K + uint64_t(k) * gpf + gi) * kAccStride;
            uint32_t backoff = kMinBackoff;
            while (((v = ld_relaxed(p)) >> 40) != 32) {
              resolver_pause(backoff);
            }
            v &= (1ull << 40) - 1;
          }
          prefix += warp_sum_u64(v);
        }
        const uint32_t jj = j - 32 * g;  // earlier tiles of this group
        uint64_t v = 0;
        if (uint32_t(lane) < jj) {
          const uint64_t* p = sc.status + uint64_t(t - jj + lane) * kStatusStride;
          uint64_t st;
          uint32_t backoff = kMinBackoff;
          while (status_flag(st = ld_relaxed(p), epoch) == 0) {
            resolver_pause(backoff);
          }
          v = status_value(st);
        }
        prefix += warp_sum_u64(v);
      }
      if (lane == 0) {
        if (j != 0) {
          uint64_t a;
          uint32_t backoff = kMinBackoff;
          while (status_flag(a = ld_relaxed(sc.aux + k), epoch) != kFlagP) {
            resolver_pause(backoff);
          }
          fstart = status_value(a);
        }
        excl = fstart + a16(4 * nwords_k) + uint64_t(G::W) * prefix;
      }
      if (lane == 0) {
        ZPROF_ADD(3, clock64() - c1);
        s_off[s] = excl;
        s_fs[s] = fstart;
        if (!kNamedBars) mbar_arrive(&bar_off[s]);
      }
      __syncwarp();
      if (kNamedBars) named_arrive(kBarOff0 + s, 32 * (CW + 1));
    }
  } else {
  // ------------------------------------------------------------------------- consumers
  // CW warps, warp w owns slab w (PW elements = PW/32 rows of 32 words) of every tile.
  // count(i):   rows -> one ballot per row = one bitmap word (fp32) / two ballots (16-bit);
  //             slab totals; the tile count is published (A) and added to the accumulators.
  // emit(i-1):  wait for tile i-1's offset, re-read its rows from the stage and store every
  //             non-zero straight to global memory at its rank (a warp's predicated 4-byte
  //             stores of one row cover a contiguous range); store the slab's bitmap words.
  // count(i) runs before emit(i-LAG), so a tile's count never waits for an older tile's offset.
  const uint32_t lt = (1u << lane) - 1u;
  auto consumer_sync = [] { asm volatile("bar.sync 1, %0;" ::"n"(32 * CW) : "memory"); };
  // element e of the tile: from the stage (bulk-copied part), the global tail, or zero
  auto load_elem = [&](auto full_tag, const uint8_t* stage, const T* gsrc, uint32_t e, uint32_t te, uint32_t be) {
    constexpr bool full = decltype(full_tag)::value;
    if (full) return uint32_t(reinterpret_cast<const T*>(stage)[e]);
    return e < be ? uint32_t(reinterpret_cast<const T*>(stage)[e]) : (e < te ? uint32_t(gsrc[e]) : 0u);
  };
  constexpr int EROWS = PW / 32;  // rows of 32 elements per slab
  auto group_wait = [&](uint64_t* bar, uint32_t parity) {  // one warp polls, the rest block in bar.sync
    if (warp == 0) {
      if (CSWAP_ZVC_CWAIT) mbar_wait(bar, parity);
      else mbar_wait_sleep(bar, parity, kConsumerSleep);
    }
    consumer_sync();
    if (warp != 0) mbar_wait(bar, parity);  // phase already complete: returns at once
  };

  auto count_slab = [&](auto full_tag, uint8_t* stage, const T* gsrc, uint32_t te, uint32_t be,
                        uint32_t* bm_out) {
    // row m = elements [32m, 32m+32) of the slab: one ballot is bitmap word (slab word m); the
    // non-zeros are compacted in place to the start of the slab (a row's writes land at or
    // before the row, and every row of a batch is loaded before any of its writes).
    // Rows go in batches of 4 (CSWAP_ZVC_BATCH) so the batch's loads issue back to back.
    constexpr int B = EROWS < CSWAP_ZVC_BATCH ? EROWS : CSWAP_ZVC_BATCH;
    const uint32_t e0 = warp * PW + lane;
    T* sv = reinterpret_cast<T*>(stage) + warp * PW;
    // shared byte address of the next compacted slot, so a lane's store address is one shift-add
    // (an element index costs an add and a scaled add per row)
    const uint32_t sdp0 = uint32_t(__cvta_generic_to_shared(sv));
    uint32_t sdp = sdp0;
    uint32_t v[B], vn[B];
#pragma unroll
    for (int u = 0; u < B; u++) v[u] = load_elem(full_tag, stage, gsrc, e0 + 32 * u, te, be);
#pragma unroll
    for (int m0 = 0; m0 < EROWS; m0 += B) {
      uint32_t wq[4];
      static_assert(B % 4 == 0, "bitmap words are stored in fours");
      // the batch's compaction stores may overwrite words other lanes just loaded: order every
      // lane's loads before any lane's stores (a ballot synchronises but does not order memory)
      __syncwarp();
      // software pipelining: the next batch's loads issue before this batch's stores (those land
      // at or before this batch's rows, never in the next batch's)
      if (CSWAP_ZVC_PF && m0 + B < EROWS) {
#pragma unroll
        for (int u = 0; u < B; u++) vn[u] = load_elem(full_tag, stage, gsrc, e0 + 32 * (m0 + B + u), te, be);
      }
#pragma unroll
      for (int u = 0; u < B; u++) {
        uint32_t w;
        if (CSWAP_ZVC_ROWASM) {
          // one predicate for the ballot and the store (written in C++, ptxas recomputes the
          // row's predicate for the predicated store)
          row_compact<T>(v[u], lt, sdp, w);
        } else {
          w = __ballot_sync(0xffffffffu, v[u] != 0);
        }
        // bitmap words leave lane 0 four at a time (one 16-byte shared store per 4 rows)
        if (CSWAP_ZVC_BM4) {
          wq[u & 3] = w;
          if ((u & 3) == 3 && lane == 0)
            *reinterpret_cast<uint4*>(bm_out + m0 + u - 3) = make_uint4(wq[0], wq[1], wq[2], wq[3]);
        } else if (lane == 0) {
          bm_out[m0 + u] = w;
        }
        if (!CSWAP_ZVC_ROWASM) {
          if (v[u]) sts_word<T>(mad_u32<G::W>(__popc(w & lt), sdp), v[u]);
          sdp = mad_u32<G::W>(__popc(w), sdp);
        }
      }
      if (m0 + B < EROWS) {
        if (!CSWAP_ZVC_PF) {
          __syncwarp();  // this batch's stores before the next batch's loads
#pragma unroll
          for (int u = 0; u < B; u++) vn[u] = load_elem(full_tag, stage, gsrc, e0 + 32 * (m0 + B + u), te, be);
        }
#pragma unroll
        for (int u = 0; u < B; u++) v[u] = vn[u];
      }
    }
    __syncwarp();
    return (sdp - sdp0) / G::W;
  };

  // copy the slab's compacted non-zeros (count_slab) to the container (emit_words)
  auto emit_slab = [&](const uint8_t* stage, uint32_t cnt, uint8_t* dst) {
    emit_words<T>(reinterpret_cast<const T*>(stage) + warp * PW, cnt, dst, lane, 32);
  };

  auto count = [&](uint32_t i, uint32_t t) {
    const int s = i % S;
    uint32_t k, j, te, be;
    uint64_t Fk;
    tile_geom(t, k, j, Fk, te, be);
    const T* gsrc = in + uint64_t(k) * F + uint64_t(j) * G::TILE;
    uint8_t* stage = s_in + s * TB;
    uint32_t* bm_out = s_bm + s * G::WT + warp * WPW;
    const uint32_t c = (te == G::TILE && be == G::TILE) ? count_slab(std::true_type{}, stage, gsrc, te, be, bm_out)
                                                        : count_slab(std::false_type{}, stage, gsrc, te, be, bm_out);
    if (lane == 0) s_wtot[s][warp] = c;
    consumer_sync();
    if (tid == 0) {  // publish the tile count (A) and feed the group accumulator
      uint32_t tot = 0;
#pragma unroll
      for (int w = 0; w < CW; w++) tot += s_wtot[s][w];
      st_relaxed(sc.status + uint64_t(t) * kStatusStride, make_status(tot, epoch, kFlagA));  // self-contained: no release needed
      if (CSWAP_ZVC_FRAMEACC) atomicAdd(reinterpret_cast<unsigned long long*>(sc.zacc + k * kAccStride), (1ull << 40) + tot);
      atomicAdd(reinterpret_cast<unsigned long long*>(sc.zacc + (K + uint64_t(k) * gpf + j / 32) * kAccStride),
                (1ull << 40) + tot);
      s_nnz[s] = tot;
      if (!kNamedBars) mbar_arrive(&bar_cnt[s]);
    }
    if (kNamedBars && warp == 0) {
      __syncwarp();
      named_arrive(kBarCnt0 + s, 64);
    }
  };

  auto emit = [&](uint32_t i, uint32_t t) {
    const int s = i % S;
    long long c0 = clock64();
    if (kNamedBars) named_sync(kBarOff0 + s, 32 * (CW + 1));
    else group_wait(&bar_off[s], (i / S) & 1);
    if (tid == 0) ZPROF_ADD(5, clock64() - c0);
    long long c2 = clock64();
    const uint64_t g0 = s_off[s], fstart = s_fs[s];
    uint32_t k, j, te, be;
    uint64_t Fk;
    tile_geom(t, k, j, Fk, te, be);
    const uint8_t* stage = s_in + s * TB;
    uint32_t woff = 0, nnz = 0;
#pragma unroll
    for (int w = 0; w < CW; w++) {
      const uint32_t x = s_wtot[s][w];
      woff += w < warp ? x : 0;
      nnz += x;
    }
    uint8_t* dst = out + g0 + uint64_t(G::W) * woff;
    emit_slab(stage, s_wtot[s][warp], dst);
    {  // this slab's bitmap words, clipped to the frame's bitmap section (incl. its 16-byte pad)
      const uint64_t wsec = (cdiv(Fk, 32) + 3) & ~uint64_t(3);
      const uint64_t w0 = uint64_t(j) * G::WT + warp * WPW;
      if (w0 < wsec) {
        const uint32_t nv = uint32_t((umin64(w0 + WPW, wsec) - w0) / 4);
        uint4* bdst = reinterpret_cast<uint4*>(out + fstart + 4 * w0);
        const uint4* bsrc = reinterpret_cast<const uint4*>(s_bm + s * G::WT + warp * WPW);
        if (uint32_t(lane) < nv) stg_stream(bdst + lane, bsrc[lane]);
      }
    }
    const uint64_t g1 = g0 + uint64_t(nnz) * G::W;
    if (warp == CW - 1 && lane == 31) {
      if (uint64_t(j) * G::TILE + G::TILE >= Fk) {  // last tile of the frame: pad + frame_bytes[k]
        for (uint64_t b = g1; b < a16(g1); b += 2) *reinterpret_cast<uint16_t*>(out + b) = 0;
        *reinterpret_cast<uint64_t*>(out + 64 + 8ull * k) = a16(g1) - fstart;
      }
      if (t == num_tiles - 1) {
        const uint64_t total = a16(g1);
        write_header(out, kZVC, dtype, n, F, K, 0, total);
        for (uint64_t b = 64 + 8ull * K; b < data_start(K); b += 8) *reinterpret_cast<uint64_t*>(out + b) = 0;
        *out_size = total;
      }
    }
    // the stage is released only after every store of this warp's part of the tile, the frame's
    // pad and frame-table entry included: the producer counts the tile as emitted on this
    // barrier and may then publish the frame (swap-out progress) with that entry
    __syncwarp();
    if (lane == 0) mbar_arrive(&bar_empty[s]);
    if (tid == 0) ZPROF_ADD(6, clock64() - c2);
  };

  // a pending tile's ticket stays in s_ticket[its stage] until its emit releases the stage
  for (uint32_t i = 0;; i++) {
    const int s = i % S;
    long long c0 = clock64();
    group_wait(&bar_full[s], (i / S) & 1);
    if (tid == 0) ZPROF_ADD(7, clock64() - c0);
    const uint32_t t = s_ticket[s];
    if (t == SENT) {
      for (uint32_t p = i > uint32_t(LAG) ? i - LAG : 0; p < i; p++) emit(p, s_ticket[p % S]);
      // every pending tile is resolved (its resolver has read s_nnz): now stop the resolvers
      if (tid == 0) {
        for (uint32_t i2 = i; i2 < i + S; i2++) {
          s_nnz[i2 % S] = SENT;
          if (!kNamedBars) mbar_arrive(&bar_cnt[i2 % S]);
        }
      }
      if (kNamedBars && warp == 0) {
        __syncwarp();
        for (int s2 = 0; s2 < S; s2++) named_arrive(kBarCnt0 + s2, 64);
      }
      break;
    }
    long long c3 = clock64();
    count(i, t);
    if (tid == 0) ZPROF_ADD(8, clock64() - c3);
    if (i >= uint32_t(LAG)) emit(i - LAG, s_ticket[(i - LAG) % S]);
  }
  }  // consumers

  // The accumulators clean up after themselves (no zero-fill launch before the kernel): the
  // last CTA to finish zeroes every accumulator word this launch used, so the next compress on
  // this scratch block (stream-ordered after this one) starts from zeros.  sc.zacc is used by
  // the persistent compress only; it is zeroed when the block is allocated.
  __syncthreads();
  __shared__ uint32_t s_last;
  const uint64_t nacc = 2 * uint64_t(K) + uint64_t(K) * gpf;
  if (tid == 0) {
    unsigned long long old;
    asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], 1;" : "=l"(old) : "l"(sc.zacc + nacc * kAccStride) : "memory");
    s_last = old + 1 == gridDim.x;
  }
  __syncthreads();
  if (s_last) {
    if (sc.kclock && tid == 0) sc.kclock[1] = globaltimer_ns();  // before the host-memory stores below
    for (uint64_t q = tid; q < nacc; q += blockDim.x) sc.zacc[q * kAccStride] = 0;
    if (tid == 0) sc.zacc[nacc * kAccStride] = 0;
    // swap-out progress published at the end (prog_mode 2): every tile of every CTA is emitted
    // (each CTA's done-count release covers its stores; this CTA acquired all of them), so the
    // frame starts and frame-table entries are final
    if (sc.prog && sc.prog_mode == 2)
      for (uint32_t k = tid; k < K; k += blockDim.x)
        publish_frame(sc.prog, k, status_value(ld_relaxed(sc.aux + k)) +
                                      ld_relaxed(reinterpret_cast<const uint64_t*>(out + 64) + k));
  }
}

// ------------------------------------------------------------------------------------------
// decompress: counts -> per-frame scan -> expand
// ------------------------------------------------------------------------------------------
// One warp per tile: popcount of the tile's bitmap slice; checks the bits past the frame end.
template <typename T>
__global__ void __launch_bounds__(kThreads) zvc_count_kernel(const uint8_t* __restrict__ in, uint64_t n, uint64_t F,
                                                             uint32_t tpf, uint32_t k0, uint32_t num_tiles,
                                                             Scratch sc, uint32_t* err) {
  using G = ZvcGeom<T>;
  const int lane = threadIdx.x & 31;
  const uint32_t tl = blockIdx.x * kWarps + (threadIdx.x >> 5);
  if (CSWAP_PDL_TRIGGER) pdl_trigger();
  pdl_wait();  // prep's frame starts / sizes and error word
  if (tl >= num_tiles || *reinterpret_cast<volatile const uint32_t*>(err)) return;
  const uint32_t t = tl + k0 * tpf;
  const uint32_t k = t / tpf, j = t % tpf;
  const uint64_t Fk = frame_len(n, F, k);
  const uint32_t tile_elems = uint32_t(umin64(G::TILE, Fk - uint64_t(j) * G::TILE));
  const uint32_t nw = (tile_elems + 31) / 32;
  const uint64_t fstart = sc.aux[k], fbytes = sc.aux2[k];
  if (a16(4 * cdiv(Fk, 32)) > fbytes) {
    if (lane == 0) set_error(err, kErrCorrupt);
    return;
  }
  const uint32_t* bm = reinterpret_cast<const uint32_t*>(in + fstart) + uint64_t(j) * G::WT;
  uint32_t c = 0;
  if (tile_elems == uint32_t(G::TILE)) {  // full tile: all 16-byte loads issued back to back
    constexpr int V = G::WT / 128;        // uint4 per lane (2 for f32, 4 for 16-bit)
    uint4 v[V];
#pragma unroll
    for (int i = 0; i < V; i++) v[i] = __ldg(reinterpret_cast<const uint4*>(bm) + i * 32 + lane);
#pragma unroll
    for (int i = 0; i < V; i++) c += __popc(v[i].x) + __popc(v[i].y) + __popc(v[i].z) + __popc(v[i].w);
    c = __reduce_add_sync(0xffffffffu, c);
    if (lane == 0) sc.tbuf[t] = c;
    return;
  }
  for (uint32_t w = lane; w < nw; w += 32) {
    uint32_t x = bm[w];
    if (w == nw - 1 && (tile_elems & 31)) {
      const uint32_t keep = (1u << (tile_elems & 31)) - 1;
      if (x & ~keep) set_error(err, kErrCorrupt);
      x &= keep;
    }
    c += __popc(x);
  }
  c = __reduce_add_sync(0xffffffffu, c);
  if (lane == 0) sc.tbuf[t] = c;
}

// One CTA per frame: exclusive scan of tile counts -> absolute value offsets; validates the
// frame size against the header's frame table.
template <typename T>
__global__ void __launch_bounds__(1024) zvc_scan_kernel(uint64_t n, uint64_t F, uint32_t tpf, uint32_t k0, Scratch sc,
                                                        uint32_t* err) {
  using G = ZvcGeom<T>;
  __shared__ uint64_t s_w[33];
  if (CSWAP_PDL_TRIGGER) pdl_trigger();
  pdl_wait();  // the count kernel's tile counts
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const uint32_t k = k0 + blockIdx.x;
  const uint64_t Fk = frame_len(n, F, k);
  const uint32_t nt = uint32_t(cdiv(Fk, G::TILE));
  const uint64_t base = sc.aux[k] + a16(4 * cdiv(Fk, 32));
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t carry = 0;
  for (uint32_t c0 = 0; c0 < nt; c0 += blockDim.x) {
    const uint32_t j = c0 + threadIdx.x;
    const uint64_t v = j < nt ? sc.tbuf[uint64_t(k) * tpf + j] : 0;
    uint64_t inc = v;
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
    if (j < nt) sc.tbuf[uint64_t(k) * tpf + j] = base + G::W * (carry + s_w[warp] + inc - v);
    carry += s_w[32];
    __syncthreads();
  }
  if (threadIdx.x == 0 && a16(4 * cdiv(Fk, 32)) + a16(G::W * carry) != sc.aux2[k]) set_error(err, kErrCorrupt);
}

template <typename T>
__global__ void __launch_bounds__(kThreads) zvc_expand_kernel(const uint8_t* __restrict__ in, T* __restrict__ outp,
                                                              uint64_t n, uint64_t F, uint32_t tpf, uint32_t k0,
                                                              Scratch sc, uint32_t* err) {
  using G = ZvcGeom<T>;
  __shared__ __align__(8) uint64_t s_bar;
  __shared__ __align__(16) uint32_t s_bm[G::WT + 4];
  __shared__ uint32_t s_pre[G::WT];  // full tiles: non-zeros of the tile before bitmap word i
  __shared__ uint32_t s_woff[kWarps];
  extern __shared__ __align__(16) uint8_t s_val[];  // kTileBytes + 32
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t t = blockIdx.x + k0 * tpf;
  const uint32_t k = t / tpf, j = t % tpf;
  const uint64_t Fk = frame_len(n, F, k);
  const uint32_t tile_elems = uint32_t(umin64(G::TILE, Fk - uint64_t(j) * G::TILE));
  const uint32_t nw = (tile_elems + 31) / 32;
  pdl_wait();  // the scan kernel's value offsets
  if (*reinterpret_cast<volatile const uint32_t*>(err)) return;
  const uint64_t fstart = sc.aux[k], fend = fstart + sc.aux2[k];
  const uint64_t vbeg = sc.tbuf[t];
  const uint64_t vend = (j + 1 < uint32_t(cdiv(Fk, G::TILE))) ? sc.tbuf[t + 1] : 0;  // next tile's start
  // Both bulk copies are issued at once (one round trip): the bitmap slice, and the value span
  // known from the scanned offsets alone — [this tile's offset, next tile's offset), or up to
  // the frame end for the frame's last tile (an aligned superset inside the container).
  const uint32_t bm_bytes = ((nw * 4) + 15) & ~15u;
  const uint8_t* bsrc = in + fstart + uint64_t(j) * G::WT * 4;
  const uint64_t abeg = vbeg & ~uint64_t(15);
  const uint64_t aend = vend ? a16(vend) : fend;
  const uint32_t d = uint32_t(vbeg - abeg);
  const bool span_ok = vbeg >= fstart && aend <= fend && aend >= abeg && aend - abeg <= kTileBytes + 32;
  if (tid == 0) {
    mbar_init(&s_bar, 1);
    const uint32_t vbytes = span_ok ? uint32_t(aend - abeg) : 0;
    mbar_expect_tx(&s_bar, bm_bytes + vbytes);
    bulk_g2s(s_bm, bsrc, bm_bytes, &s_bar);
    if (vbytes) bulk_g2s(s_val, in + abeg, vbytes, &s_bar);
  }
  __syncthreads();
  mbar_wait(&s_bar, 0);
  T* dst = outp + uint64_t(k) * F + uint64_t(j) * G::TILE;
  if (tile_elems == uint32_t(G::TILE)) {
    // ---- full tile (every tile but a frame's last): per-word exclusive prefix table, then per
    // lane one bitmap word + one prefix load per 16-byte output vector (no per-word loops)
    constexpr int WPT = G::WT / kThreads;  // bitmap words per thread for the table (1 or 2)
    static_assert(WPT >= 1 && WPT * kThreads == G::WT, "expand geometry");
    uint32_t pc[WPT], c = 0;
#pragma unroll
    for (int i = 0; i < WPT; i++) {
      pc[i] = __popc(s_bm[tid * WPT + i]);
      c += pc[i];
    }
    uint32_t inc = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
    if (lane == 31) s_woff[warp] = inc;
    __syncthreads();
    uint32_t base = 0, nnz = 0;
#pragma unroll
    for (int w = 0; w < kWarps; w++) {
      const uint32_t x = s_woff[w];
      base += w < warp ? x : 0;
      nnz += x;
    }
    uint32_t run = base + inc - c;
#pragma unroll
    for (int i = 0; i < WPT; i++) {
      s_pre[tid * WPT + i] = run;
      run += pc[i];
    }
    __syncthreads();
    const uint64_t vlast = vbeg + uint64_t(nnz) * G::W;
    const bool ok = span_ok && (vend ? vend == vlast : a16(vlast) <= fend);
    if (!ok && tid == 0) set_error(err, kErrCorrupt);
    const uint32_t sv = uint32_t(__cvta_generic_to_shared(s_val)) + d;  // shared address of value 0
#pragma unroll 2
    for (int q = 0; q < G::NCH; q++) {
      const uint32_t e0 = warp * G::PER_WARP + q * G::CHUNK + lane * G::EPV;
      const uint32_t wi = e0 >> 5, sh = e0 & 31;
      const uint32_t mine = s_bm[wi];
      uint32_t a = sv + G::W * (s_pre[wi] + __popc(mine & ((1u << sh) - 1u)));
      const uint32_t b = mine >> sh;
      uint32_t w4[4];
#pragma unroll
      for (int e = 0; e < G::EPV; e++) {
        const bool on = (b >> e) & 1u;
        uint32_t x = 0;
        if constexpr (sizeof(T) == 4) {
          if (on) x = lds_u32(a);
          w4[e] = x;
        } else {
          if (on) x = lds_u16(a);
          if (e & 1) w4[e >> 1] |= x << 16;
          else w4[e >> 1] = x;
        }
        a += on ? G::W : 0;
      }
      if (!ok) w4[0] = w4[1] = w4[2] = w4[3] = 0;
      stg_stream(reinterpret_cast<uint4*>(dst + e0), make_uint4(w4[0], w4[1], w4[2], w4[3]));
    }
    return;
  }
  // ---- a frame's short last tile: bounds-checked general path
  {
    constexpr int WPW = G::WT / kWarps;
    uint32_t c = 0;
#pragma unroll
    for (int i = 0; i < WPW / 32; i++) {
      const uint32_t wi = warp * WPW + i * 32 + lane;
      uint32_t x = wi < nw ? s_bm[wi] : 0;
      if (wi == nw - 1 && (tile_elems & 31)) x &= (1u << (tile_elems & 31)) - 1;
      c += __popc(x);
    }
    c = __reduce_add_sync(0xffffffffu, c);
    if (lane == 0) s_woff[warp] = c;
  }
  __syncthreads();
  uint32_t woff = 0, nnz = 0;
#pragma unroll
  for (int w = 0; w < kWarps; w++) {
    woff += w < warp ? s_woff[w] : 0;
    nnz += s_woff[w];
  }
  const uint64_t vlast = vbeg + uint64_t(nnz) * G::W;
  const bool ok = span_ok && (vend ? vend == vlast : a16(vlast) <= fend);
  if (!ok && tid == 0) set_error(err, kErrCorrupt);
  uint32_t r = woff;
#pragma unroll 1
  for (int q = 0; q < G::NCH; q++) {
    const uint32_t e0 = warp * G::PER_WARP + q * G::CHUNK + lane * G::EPV;
    const uint32_t cw0 = (warp * G::PER_WARP + q * G::CHUNK) / 32;
    const uint32_t myw = e0 / 32;
    uint32_t before = 0, mine = 0, total = 0;
#pragma unroll
    for (int m = 0; m < G::EPV; m++) {
      const uint32_t wi = cw0 + m;
      uint32_t x = wi < nw ? s_bm[wi] : 0;
      if (wi == nw - 1 && (tile_elems & 31)) x &= (1u << (tile_elems & 31)) - 1;
      const uint32_t p = __popc(x);
      before += wi < myw ? p : 0;
      if (wi == myw) mine = x;
      total += p;
    }
    const uint32_t sh = (lane % G::LPW) * G::EPV;
    const uint32_t b = (mine >> sh) & ((1u << G::EPV) - 1);
    uint32_t rank = r + before + __popc(mine & ((1u << sh) - 1));
    uint32_t w4[4] = {0, 0, 0, 0};
#pragma unroll
    for (int e = 0; e < G::EPV; e++) {
      if ((b >> e) & 1) {
        uint32_t x;
        if constexpr (sizeof(T) == 4) x = *reinterpret_cast<const uint32_t*>(s_val + d + 4 * rank);
        else x = *reinterpret_cast<const uint16_t*>(s_val + d + 2 * rank);
        if constexpr (sizeof(T) == 4) w4[e] = x;
        else w4[e >> 1] |= x << ((e & 1) * 16);
        rank++;
      }
    }
    r += total;
    if (!ok) w4[0] = w4[1] = w4[2] = w4[3] = 0;
    if (e0 + G::EPV <= tile_elems) {
      stg_stream(reinterpret_cast<uint4*>(dst + e0), make_uint4(w4[0], w4[1], w4[2], w4[3]));
    } else {
      for (int e = 0; e < G::EPV; e++)
        if (e0 + e < tile_elems) {
          if constexpr (sizeof(T) == 4) dst[e0 + e] = w4[e];
          else dst[e0 + e] = T((w4[e >> 1] >> ((e & 1) * 16)) & 0xFFFFu);
        }
    }
  }
}

// ------------------------------------------------------------------------------------------
uint32_t zvc_tiles(uint64_t n, int w, uint64_t F, uint32_t k0, uint32_t k1, uint32_t* tpf_out) {
  const uint32_t TILE = kTileBytes / w;
  const uint32_t tpf = uint32_t(cdiv(F, TILE));
  if (tpf_out) *tpf_out = tpf;
  if (k1 <= k0) return 0;
  return (k1 - 1 - k0) * tpf + uint32_t(cdiv(frame_len(n, F, k1 - 1), TILE));
}

static std::atomic<uint32_t> g_zvc_grid{0};
static std::atomic<int> g_zvc_variant{-1};

static int prof_enabled() {
  static int p = -1;
  if (p < 0) p = getenv("CSWAP_ZVC_PROF") ? 1 : 0;
  return p;
}

// CSWAP_ZVC_COOP=0 launches the persistent compress non-cooperatively (A/B measurements only:
// without it the kernel can stall behind concurrent kernels)
static bool coop_enabled() {
  static int c = -1;
  if (c < 0) {
    const char* e = getenv("CSWAP_ZVC_COOP");
    c = (e && e[0] == '0') ? 0 : 1;
  }
  return c == 1;
}

static int sm_count() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  return sms;
}

template <typename T, int S, int CW, int TB>
static cudaError_t launch_compress_s(const void* in, uint64_t n, uint64_t F, uint8_t* out, uint64_t* out_size,
                                     const Scratch& sc, uint32_t epoch, int dtype, cudaStream_t st) {
  using L = CompressSmem<T, S, TB>;
  const uint32_t K = uint32_t(cdiv(n, F));
  const uint32_t TILE = TB / sizeof(T);
  const uint32_t tpf = uint32_t(cdiv(F, TILE));
  const uint32_t tiles = (K - 1) * tpf + uint32_t(cdiv(frame_len(n, F, K - 1), TILE));
  auto kern = zvc_compress_persistent<T, S, CW, TB>;
  constexpr int threads = compress_threads<S, CW>();
  static int per_sm = 0;  // resident CTAs per SM, from the occupancy calculator (not the estimate)
  if (!per_sm) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, L::bytes);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, threads, L::bytes) != cudaSuccess || per_sm < 1)
      return cudaErrorInvalidConfiguration;
  }
  const uint32_t cap = uint32_t(sm_count()) * uint32_t(per_sm);  // co-resident maximum
  const uint32_t want = g_zvc_grid.load(std::memory_order_relaxed);
  const uint32_t grid = std::min<uint32_t>(tiles, want ? std::min(want, cap) : cap);
  timing_kernel_start(st);
  // Forward progress: a tile waits for the COUNTS of earlier tiles, which other CTAs produce, so
  // every CTA of the grid must be resident at once.  A cooperative launch guarantees that (the
  // grid is admitted only when all of it fits), also while other kernels occupy part of the GPU
  // or a second compress runs on another stream (tests/test_gpu_concurrency.py).
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = L::bytes;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = coop_enabled() ? 1 : 0;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  const cudaError_t e = cudaLaunchKernelEx(&cfg, kern, static_cast<const T*>(in), n, F, K, tpf, tiles, out, out_size,
                                           sc, epoch, dtype, prof_enabled());
  if (e != cudaSuccess) return e;
  if (prof_enabled()) {
    unsigned long long h[16];
    cudaStreamSynchronize(st);
    cudaMemcpyFromSymbol(h, g_zprof, sizeof(h));
    fprintf(stderr,
            "[zprof] TB=%d S=%d CW=%d grid=%u tiles=%u | per-tile cycles: producer_wait_empty=%.0f "
            "resolver_wait_cnt=%.0f resolver_lookback=%.0f | consumer(tid0): wait_off=%.0f finish=%.0f "
            "wait_full=%.0f prep=%.0f\n",
            TB, S, CW, grid, tiles, h[0] / double(tiles), h[2] / double(tiles), h[3] / double(tiles),
            h[5] / double(tiles), h[6] / double(tiles), h[7] / double(tiles), h[8] / double(tiles));
    memset(h, 0, sizeof(h));
    cudaMemcpyToSymbol(g_zprof, h, sizeof(h));
  }
  return cudaGetLastError();
}

// compress configuration (stages x tile bytes): cswap_set_zvc_launch, else CSWAP_ZVC_CFG, else 0
constexpr int kMaxVariant = 9;
static int compress_cfg() {
  const int v = g_zvc_variant.load(std::memory_order_relaxed);
  if (v >= 0) return v;
  static int c = -1;
  if (c < 0) {
    const char* e = getenv("CSWAP_ZVC_CFG");
    c = e ? atoi(e) : 0;
    if (c < 0 || c > kMaxVariant) c = 0;
  }
  return c;
}

bool zvc_set_launch(uint32_t grid, int variant) {
  if (variant < -1 || variant > kMaxVariant) return false;
  g_zvc_grid.store(grid);
  g_zvc_variant.store(variant);
  return true;
}

template <typename T>
static cudaError_t launch_compress_t(const void* in, uint64_t n, uint64_t F, uint8_t* out, uint64_t* out_size,
                                     const Scratch& sc, uint32_t epoch, int dtype, cudaStream_t st) {
  switch (compress_cfg()) {
    case 1: return launch_compress_s<T, 6, 8, 16384>(in, n, F, out, out_size, sc, epoch, dtype, st);
    case 2: return launch_compress_s<T, 5, 8, 16384>(in, n, F, out, out_size, sc, epoch, dtype, st);
    case 3: return launch_compress_s<T, 4, 8, 16384>(in, n, F, out, out_size, sc, epoch, dtype, st);
    // one CTA per SM with 16 consumer warps and a deeper ring (LAG = S - 2 tile periods of slack
    // for the offsets, which wait for every earlier tile's count)
    case 4: return launch_compress_s<T, 6, 16, 32768>(in, n, F, out, out_size, sc, epoch, dtype, st);
    case 5: return launch_compress_s<T, 5, 16, 32768>(in, n, F, out, out_size, sc, epoch, dtype, st);
    case 6: return launch_compress_s<T, 4, 16, 32768>(in, n, F, out, out_size, sc, epoch, dtype, st);
    // more, smaller CTAs per SM: 4 consumer warps per 16 KiB tile, so per-tile latencies
    // (barriers, the offset wait) of 3-4 resident tiles overlap
    case 7: return launch_compress_s<T, 3, 4, 16384>(in, n, F, out, out_size, sc, epoch, dtype, st);
    case 8: return launch_compress_s<T, 4, 4, 16384>(in, n, F, out, out_size, sc, epoch, dtype, st);
    // the same 96 KiB of stages as 4 x 24 KiB: LAG = 2 tile periods for the offset to resolve
    // (the default's consumers wait ~1000-1300 cycles per tile for it, CSWAP_ZVC_PROF)
    case 9: return launch_compress_s<T, 4, 8, 24576>(in, n, F, out, out_size, sc, epoch, dtype, st);
    default: return launch_compress_s<T, 3, 8, 32768>(in, n, F, out, out_size, sc, epoch, dtype, st);
  }
}

// scratch a compress launch needs: tile status words and (frame + 32-tile group) accumulators,
// sized for the smallest compress tile any configuration uses (16 KiB)
void zvc_compress_scratch(uint64_t n, int w, uint64_t F, uint64_t* tiles, uint64_t* aux) {
  const uint64_t TILE = 16384 / w, K = cdiv(n, F), tpf = cdiv(F, TILE);
  *tiles = (K ? (K - 1) * tpf + cdiv(frame_len(n, F, K - 1), TILE) : 0) * kStatusStride;
  // sc.zacc: frame + group accumulators, fdone, CTA counter, kAccStride words apart
  *aux = (2 * K + K * ((tpf + 31) / 32) + 2) * kAccStride;
}

cudaError_t launch_zvc_compress(const void* in, uint64_t n, int w, uint64_t F, uint8_t* out, uint64_t* out_size,
                                const Scratch& sc, uint32_t epoch, int dtype, cudaStream_t st) {
  return w == 4 ? launch_compress_t<uint32_t>(in, n, F, out, out_size, sc, epoch, dtype, st)
                : launch_compress_t<uint16_t>(in, n, F, out, out_size, sc, epoch, dtype, st);
}

template <typename T>
static cudaError_t launch_zvc_decompress_t(const uint8_t* in, void* out, uint64_t n, uint64_t F, uint32_t k0,
                                           uint32_t k1, const Scratch& sc, uint32_t epoch, uint32_t* err,
                                           cudaStream_t st) {
  (void)epoch;  // the split decode needs no inter-CTA status words
  uint32_t tpf;
  const uint32_t tiles = zvc_tiles(n, sizeof(T), F, k0, k1, &tpf);
  if (!tiles) return cudaSuccess;
  timing_kernel_start(st);
  const int smem = kTileBytes + 32;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(zvc_expand_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  // programmatic dependent launch: each kernel of the chain may be launched while its
  // predecessor's last CTAs drain, and waits (griddepcontrol.wait) before reading its outputs
  CUDA_TRY_LAUNCH(pdl_launch(zvc_count_kernel<T>, dim3((tiles + kWarps - 1) / kWarps), dim3(kThreads), 0, st, in, n,
                             F, tpf, k0, tiles, sc, err));
  CUDA_TRY_LAUNCH(pdl_launch(zvc_scan_kernel<T>, dim3(k1 - k0), dim3(1024), 0, st, n, F, tpf, k0, sc, err));
  CUDA_TRY_LAUNCH(pdl_launch(zvc_expand_kernel<T>, dim3(tiles), dim3(kThreads), smem, st, in, static_cast<T*>(out), n,
                             F, tpf, k0, sc, err));
  return cudaGetLastError();
}

cudaError_t launch_zvc_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t k0,
                                  uint32_t k1, const Scratch& sc, uint32_t epoch, uint32_t* err, cudaStream_t st) {
  return w == 4 ? launch_zvc_decompress_t<uint32_t>(in, out, n, F, k0, k1, sc, epoch, err, st)
                : launch_zvc_decompress_t<uint16_t>(in, out, n, F, k0, k1, sc, epoch, err, st);
}

}  // namespace cswap
