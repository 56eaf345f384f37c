// api.cu — the C ABI of include/cswap.h: runtime (streams, scratch, pools, handles), codec
// dispatch, probe + selector, and the swap-out / swap-in pipelines.
//
// Swapping executor (PAPER.md:120 §IV-A; :228 §V): compress -> offload to pinned host memory on
// an asynchronous copy stream; prefetch -> decompress.  Memory pools replace cudaMalloc /
// cudaMallocHost on the path: device staging comes from the CUDA stream-ordered
// pool (cudaMallocAsync, release threshold = unlimited), host containers from a pinned-chunk
// allocator.  Swap-in is pipelined per frame group (R7): H2D of group g+1 overlaps the
// decompression of group g.
#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <tuple>
#include <unordered_map>
#include <vector>

#include "../../include/cswap.h"
#include "common.cuh"
#include "internal.h"
#include "kernels.h"

using namespace cswap;

namespace {

thread_local std::string g_err;

cswap_status fail(cswap_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

#define CU(x)                                                                                   \
  do {                                                                                          \
    cudaError_t e_ = (x);                                                                       \
    if (e_ != cudaSuccess) {                                                                    \
      cswap_status st_ = (e_ == cudaErrorMemoryAllocation) ? CSWAP_ERR_NOMEM : CSWAP_ERR_CUDA; \
      return fail(st_, "%s:%d %s: %s", __FILE__, __LINE__, #x, cudaGetErrorString(e_));         \
    }                                                                                           \
  } while (0)

#define TRY(x)                          \
  do {                                  \
    cswap_status s_ = (x);              \
    if (s_ != CSWAP_OK) return s_;      \
  } while (0)

inline int width(int dtype) { return dtype == CSWAP_F32 ? 4 : (dtype == CSWAP_F16 || dtype == CSWAP_BF16) ? 2 : 0; }
inline uint64_t al16(uint64_t x) { return (x + 15) / 16 * 16; }

// ---------------------------------------------------------------------------------------------
// pinned host pool: chunks from cudaHostAlloc(Portable | Mapped), first-fit, coalescing frees
// ---------------------------------------------------------------------------------------------
struct PinnedPool {
  struct Chunk {
    uint8_t* base;
    uint64_t size;
    std::map<uint64_t, uint64_t> free;  // offset -> bytes
  };
  std::mutex m;
  std::vector<Chunk> chunks;
  std::unordered_map<uint8_t*, std::pair<size_t, uint64_t>> live;  // ptr -> (chunk, bytes)
  uint64_t chunk_bytes = 512ull << 20;

  static uint64_t round(uint64_t b) { return std::max<uint64_t>(256, (b + 255) / 256 * 256); }

  uint8_t* alloc(uint64_t bytes) {
    bytes = round(bytes);
    std::lock_guard<std::mutex> lk(m);
    for (size_t c = 0; c < chunks.size(); c++) {
      auto& fl = chunks[c].free;
      for (auto it = fl.begin(); it != fl.end(); ++it) {
        if (it->second >= bytes) {
          const uint64_t off = it->first, sz = it->second;
          fl.erase(it);
          if (sz > bytes) fl[off + bytes] = sz - bytes;
          uint8_t* p = chunks[c].base + off;
          live[p] = {c, bytes};
          return p;
        }
      }
    }
    const uint64_t sz = std::max(bytes, chunk_bytes);
    void* p = nullptr;
    if (cudaHostAlloc(&p, sz, cudaHostAllocPortable | cudaHostAllocMapped) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    chunks.push_back(Chunk{static_cast<uint8_t*>(p), sz, {}});
    if (sz > bytes) chunks.back().free[bytes] = sz - bytes;
    live[static_cast<uint8_t*>(p)] = {chunks.size() - 1, bytes};
    return static_cast<uint8_t*>(p);
  }
  void release_range(size_t c, uint64_t off, uint64_t bytes) {
    auto& fl = chunks[c].free;
    auto it = fl.emplace(off, bytes).first;
    auto nx = std::next(it);
    if (nx != fl.end() && it->first + it->second == nx->first) {
      it->second += nx->second;
      fl.erase(nx);
    }
    if (it != fl.begin()) {
      auto pv = std::prev(it);
      if (pv->first + pv->second == it->first) {
        pv->second += it->second;
        fl.erase(it);
      }
    }
  }
  void free(uint8_t* p) {
    if (!p) return;
    std::lock_guard<std::mutex> lk(m);
    auto it = live.find(p);
    if (it == live.end()) return;
    const size_t c = it->second.first;
    release_range(c, uint64_t(p - chunks[c].base), it->second.second);
    live.erase(it);
  }
  void shrink(uint8_t* p, uint64_t new_bytes) {  // give back the unused tail of an allocation
    std::lock_guard<std::mutex> lk(m);
    auto it = live.find(p);
    if (it == live.end()) return;
    new_bytes = round(new_bytes);
    const uint64_t old = it->second.second;
    if (new_bytes >= old) return;
    const size_t c = it->second.first;
    release_range(c, uint64_t(p - chunks[c].base) + new_bytes, old - new_bytes);
    it->second.second = new_bytes;
  }
  void destroy() {
    for (auto& c : chunks) cudaFreeHost(c.base);
    chunks.clear();
    live.clear();
  }
};

// ---------------------------------------------------------------------------------------------
// scratch blocks (lookback status, tickets, per-frame arrays) leased per operation
// ---------------------------------------------------------------------------------------------
struct Block {
  Scratch sc{};
  cudaEvent_t ev = nullptr;
  uint32_t epoch = 0;
  std::mutex m;
};

constexpr int kBlocks = 4;

struct Ctx {
  int device = -1;
  int sms = 0;
  Block blocks[kBlocks];
  std::atomic<uint32_t> rr{0};
  cudaStream_t s_d2h = nullptr, s_h2d = nullptr;
  std::mutex cfg_m;
  cswap_calib calib{};
  cswap_format fmt{};
  PinnedPool pinned;
  uint32_t* dev_err = nullptr;  // err word for cswap_decompress(err = NULL)
  std::atomic<uint64_t> launches{0};
  std::atomic<uint64_t> graph_launches{0}, graph_instantiations{0};
  uint64_t gen = 0;  // distinguishes this context from earlier init/shutdown cycles (graph caches)
  // kernel timing (cswap_set_kernel_timing)
  std::atomic<bool> timing{false};
  std::mutex tm_m;
  struct Pend {
    cudaEvent_t a, b;
    cswap_kernel_record r;
    uint64_t* stamps;  // 2 x u64 %globaltimer (mapped pinned), or null
  };
  std::vector<Pend> pend;
};

// Brackets a launch group with CUDA events on its stream when timing is enabled.
// The start event is recorded by the launcher itself, immediately before its first kernel
// (cswap::timing_kernel_start), so that host-side enqueue time on an idle stream is not counted.
struct Timer;
thread_local Timer* t_pending = nullptr;
struct Timer {
  Ctx* c;
  cudaStream_t st;
  cudaEvent_t a = nullptr, b = nullptr;
  bool started = false;
  uint64_t* stamps = nullptr;  // filled by stamp kernels first / last in the group (run_group)
  Timer(Ctx* ctx, cudaStream_t s);
  void start_now() {
    if (a && !started) {
      cudaEventRecord(a, st);
      started = true;
    }
  }
  void stop() {
    if (t_pending == this) t_pending = nullptr;
    start_now();  // no launcher marked a start: fall back to "now"
    if (a && !b && cudaEventCreate(&b) == cudaSuccess) cudaEventRecord(b, st);
  }
  void commit(int codec, int dir, uint64_t raw, uint64_t comp) {
    if (!a) return;
    stop();
    std::lock_guard<std::mutex> lk(c->tm_m);
    c->pend.push_back(Ctx::Pend{a, b, cswap_kernel_record{codec, dir, raw, comp, 0.0, 0.0}, stamps});
    a = b = nullptr;
    stamps = nullptr;
  }
  ~Timer();
};
}  // namespace

namespace {
Timer::Timer(Ctx* ctx, cudaStream_t s) : c(ctx), st(s) {
  if (c->timing.load() && cudaEventCreate(&a) == cudaSuccess) {
    t_pending = this;
    stamps = reinterpret_cast<uint64_t*>(c->pinned.alloc(16));
    if (stamps) stamps[0] = stamps[1] = 0;
  }
}
Timer::~Timer() {
  if (t_pending == this) t_pending = nullptr;
  if (a) cudaEventDestroy(a);
  if (b) cudaEventDestroy(b);
  if (stamps) c->pinned.free(reinterpret_cast<uint8_t*>(stamps));  // not committed
}
}  // namespace

void cswap::timing_kernel_start(cudaStream_t) {
  if (t_pending) t_pending->start_now();
}

namespace {

// ---------------------------------------------------------------------------------------------
// launch groups as CUDA graphs
// ---------------------------------------------------------------------------------------------
// While a copy engine streams over PCIe (the swap pipeline always has one running), every
// kernel boundary of plainly launched kernels costs 5-10 us (tools/launch_probe.py on B200:
// 2.1 us per boundary alone, 9.6 us during a D2H, 5.5 us during an H2D), while the boundaries
// inside an uploaded graph cost 0.5 us in all three cases.  So the kernels of one launch group
// (one compress; one swap-in frame group; one decompress) are captured on a per-thread capture
// stream and replayed on the caller's stream as one graph.  The executable graph is cached per
// (thread, stream, group key) and updated in place (cudaGraphExecUpdate) with the new pointers /
// sizes; it is re-instantiated only when the topology changes.  CSWAP_GRAPHS=0 launches plainly.
std::atomic<uint64_t> g_gen{0};
cswap_status cuda_status(cudaError_t e, const char* what);

bool graphs_enabled() {
  static int on = -1;
  if (on < 0) {
    const char* e = getenv("CSWAP_GRAPHS");
    on = (e && e[0] == '0') ? 0 : 1;
  }
  return on == 1;
}

struct GraphCache {
  struct Ent {
    cudaGraphExec_t exec = nullptr;
    uint64_t last = 0;
  };
  std::map<std::tuple<cudaStream_t, uint64_t>, Ent> m;
  cudaStream_t cap = nullptr;
  uint64_t gen = 0, tick = 0;
  void reset(uint64_t g) {
    if (gen == g_gen.load()) {  // the context these belong to is still alive
      for (auto& kv : m)
        if (kv.second.exec) cudaGraphExecDestroy(kv.second.exec);
      if (cap) cudaStreamDestroy(cap);
    }
    m.clear();
    cap = nullptr;
    gen = g;
  }
};
thread_local GraphCache t_gc;
constexpr size_t kGraphCacheMax = 64;

// Run fn(stream) — a function that only enqueues kernels — as one graph on st (or directly on st
// when graphs are disabled).  A pending kernel timer gets its start event on st right before the
// graph launch (timing events cannot be recorded inside a capture).
template <class Fn>
cswap_status run_group(Ctx* c, cudaStream_t st, uint64_t key, Fn&& fn) {
  Timer* pending = t_pending;
  uint64_t* stamps = pending ? pending->stamps : nullptr;
  // timed groups: stamp kernels first and last (device duration of the group)
  auto body = [&](cudaStream_t gs) -> cswap_status {
    if (stamps) {
      c->launches++;
      TRY(cuda_status(launch_stamp(stamps, gs), "stamp"));
    }
    TRY(fn(gs));
    if (stamps) {
      c->launches++;
      TRY(cuda_status(launch_stamp(stamps + 1, gs), "stamp"));
    }
    return CSWAP_OK;
  };
  if (!graphs_enabled()) {
    if (pending) pending->start_now();
    return body(st);
  }
  GraphCache& g = t_gc;
  if (g.gen != c->gen) g.reset(c->gen);
  if (!g.cap && cudaStreamCreateWithFlags(&g.cap, cudaStreamNonBlocking) != cudaSuccess)
    return fail(CSWAP_ERR_CUDA, "capture stream create failed");
  if (cudaStreamBeginCapture(g.cap, cudaStreamCaptureModeRelaxed) != cudaSuccess)
    return fail(CSWAP_ERR_CUDA, "begin capture failed: %s", cudaGetErrorString(cudaGetLastError()));
  t_pending = nullptr;
  cswap_status s = body(g.cap);
  t_pending = pending;
  cudaGraph_t graph = nullptr;
  const cudaError_t e = cudaStreamEndCapture(g.cap, &graph);
  if (s != CSWAP_OK || e != cudaSuccess) {
    if (graph) cudaGraphDestroy(graph);
    cudaGetLastError();
    return s != CSWAP_OK ? s : fail(CSWAP_ERR_CUDA, "capture failed: %s", cudaGetErrorString(e));
  }
  auto& ent = g.m[std::make_tuple(st, key)];
  ent.last = ++g.tick;
  if (ent.exec) {
    cudaGraphExecUpdateResultInfo info;
    if (cudaGraphExecUpdate(ent.exec, graph, &info) != cudaSuccess) {
      cudaGetLastError();
      cudaGraphExecDestroy(ent.exec);
      ent.exec = nullptr;
    }
  }
  if (!ent.exec) {
    if (cudaGraphInstantiate(&ent.exec, graph, 0) != cudaSuccess) {
      ent.exec = nullptr;
      cudaGraphDestroy(graph);
      return fail(CSWAP_ERR_CUDA, "graph instantiate failed: %s", cudaGetErrorString(cudaGetLastError()));
    }
    c->graph_instantiations++;
  }
  cudaGraphDestroy(graph);
  if (pending) pending->start_now();
  if (cudaGraphLaunch(ent.exec, st) != cudaSuccess)
    return fail(CSWAP_ERR_CUDA, "graph launch failed: %s", cudaGetErrorString(cudaGetLastError()));
  c->graph_launches++;
  if (g.m.size() > kGraphCacheMax) {  // evict the least recently used (freed once it has run)
    auto lru = g.m.begin();
    for (auto it = g.m.begin(); it != g.m.end(); ++it)
      if (it->second.last < lru->second.last) lru = it;
    if (lru->second.exec) cudaGraphExecDestroy(lru->second.exec);
    g.m.erase(lru);
  }
  return CSWAP_OK;
}

// group keys: kind << 16 | codec << 8 | dtype
constexpr uint64_t kGrpCompress = 1, kGrpSwapIn = 2, kGrpSwapInFirst = 3, kGrpDecompress = 4;
inline uint64_t group_key(uint64_t kind, int codec, int dtype) {
  return kind << 16 | uint64_t(codec) << 8 | uint64_t(dtype);
}

}  // namespace

namespace {

Ctx* g_ctx = nullptr;
std::mutex g_mu;
cswap_calib g_default_calib;
bool g_default_init = false;

const cswap_calib& builtin_calib() {
  if (!g_default_init) {
    default_calib(&g_default_calib);
    g_default_init = true;
  }
  return g_default_calib;
}

cswap_status ensure_block(Block& b, uint64_t tiles, uint64_t aux) {
  tiles = std::max<uint64_t>(tiles, 1024);
  aux = std::max<uint64_t>(aux, 1024);
  if (b.sc.status && b.sc.cap_tiles >= tiles && b.sc.cap_aux >= aux) return CSWAP_OK;
  if (b.ev) CU(cudaEventSynchronize(b.ev));
  if (b.sc.status) {
    cudaFree(b.sc.status);
    cudaFree(b.sc.tickets);
    cudaFree(b.sc.aux);
    cudaFree(b.sc.aux2);
    cudaFree(b.sc.err);
    cudaFree(b.sc.tbuf);
    cudaFree(b.sc.tbuf2);
    cudaFree(b.sc.aux3);
  }
  tiles = std::max(tiles, b.sc.cap_tiles * 2);
  aux = std::max(aux, b.sc.cap_aux * 2);
  CU(cudaMalloc(&b.sc.status, tiles * 8));
  CU(cudaMalloc(&b.sc.tickets, kEpochs * 4));
  CU(cudaMalloc(&b.sc.aux, aux * 8));
  CU(cudaMalloc(&b.sc.aux2, aux * 8));
  CU(cudaMalloc(&b.sc.err, 64));
  CU(cudaMalloc(&b.sc.tbuf, tiles * 8));
  CU(cudaMalloc(&b.sc.tbuf2, tiles * 32));  // 32 B per tile: CSR keeps 8 u32 slab counts
  CU(cudaMalloc(&b.sc.aux3, aux * 8));
  CU(cudaMemset(b.sc.status, 0, tiles * 8));
  // epoch-tagged words are also polled in aux (frame starts): a fresh block restarts at epoch 0,
  // so memory recycled from an earlier block could hold words tagged with a live epoch; zero
  // every scratch array once (compute-sanitizer initcheck flagged the first reads of aux)
  CU(cudaMemset(b.sc.aux, 0, aux * 8));
  CU(cudaMemset(b.sc.aux2, 0, aux * 8));
  CU(cudaMemset(b.sc.aux3, 0, aux * 8));
  CU(cudaMemset(b.sc.tbuf, 0, tiles * 8));
  CU(cudaMemset(b.sc.tbuf2, 0, tiles * 32));
  CU(cudaMemset(b.sc.tickets, 0, kEpochs * 4));
  CU(cudaMemset(b.sc.err, 0, 64));
  b.sc.cap_tiles = tiles;
  b.sc.cap_aux = aux;
  b.epoch = 0;
  return CSWAP_OK;
}

// RAII lease: the stream waits for the block's previous user; the block's event is recorded
// on the stream when the lease ends.
struct Lease {
  Block* b = nullptr;
  Ctx* ctx = nullptr;
  cudaStream_t st = nullptr;
  std::unique_lock<std::mutex> lk;
  cswap_status status = CSWAP_OK;
  Lease(Ctx& c, cudaStream_t s, uint64_t tiles, uint64_t aux) : ctx(&c), st(s) {
    const uint32_t start = c.rr.fetch_add(1);
    // prefer a free block that is already large enough: growing one (ensure_block) frees and
    // re-allocates device memory, which synchronises the device — if every block had to grow
    // in turn, each of the first kBlocks large operations would pay that (a calibration sample
    // measured 99 ms for a 256 MiB decode that way)
    for (int pass = 0; pass < 2 && !b; pass++) {
      for (int i = 0; i < kBlocks && !b; i++) {
        Block& cand = c.blocks[(start + i) % kBlocks];
        std::unique_lock<std::mutex> l(cand.m, std::try_to_lock);
        if (!l.owns_lock()) continue;
        if (pass == 0 && !(cand.sc.status && cand.sc.cap_tiles >= std::max<uint64_t>(tiles, 1024) &&
                           cand.sc.cap_aux >= std::max<uint64_t>(aux, 1024)))
          continue;
        b = &cand;
        lk = std::move(l);
      }
    }
    if (!b) {
      b = &c.blocks[start % kBlocks];
      lk = std::unique_lock<std::mutex>(b->m);
    }
    status = ensure_block(*b, tiles, aux);
    if (status == CSWAP_OK && cudaStreamWaitEvent(st, b->ev, 0) != cudaSuccess)
      status = fail(CSWAP_ERR_CUDA, "cudaStreamWaitEvent failed");
  }
  uint32_t epoch() {
    if (++b->epoch >= kEpochs) {
      launch_zero_words(b->sc.status, b->sc.cap_tiles * 2, st);
      launch_zero_words(b->sc.tickets, kEpochs, st);
      launch_zero_words(b->sc.aux, b->sc.cap_aux * 2, st);  // epoch-tagged frame starts
      ctx->launches += 3;
      b->epoch = 1;
    }
    return b->epoch;
  }
  ~Lease() {
    if (b && b->ev) cudaEventRecord(b->ev, st);
  }
};

cswap_status need_ctx(Ctx** out) {
  if (!g_ctx) return fail(CSWAP_ERR_NOT_READY, "cswap_init has not been called");
  *out = g_ctx;
  return CSWAP_OK;
}

cswap_status check_fmt(const cswap_format& f) {
  if (f.frame_elems == 0 || f.frame_elems % 1024) return fail(CSWAP_ERR_INVALID, "frame_elems must be a positive multiple of 1024");
  if (f.csr_row == 0 || f.frame_elems % f.csr_row) return fail(CSWAP_ERR_INVALID, "csr_row must divide frame_elems");
  if (f.lz4_block == 0 || f.lz4_block > 65536 || f.lz4_block % 1024)
    return fail(CSWAP_ERR_INVALID, "lz4_block must be a multiple of 1024 and <= 65536");
  return CSWAP_OK;
}

cswap_format resolve_fmt(Ctx* c, const cswap_format* f) {
  if (f) return *f;
  std::lock_guard<std::mutex> lk(c->cfg_m);
  return c->fmt;
}

uint32_t param_of(int codec, const cswap_format& f) {
  return codec == CSWAP_CODEC_CSR ? f.csr_row : codec == CSWAP_CODEC_LZ4 ? f.lz4_block : 0;
}

uint64_t max_size(uint64_t n, int w, int codec, const cswap_format& f) {
  const uint64_t F = f.frame_elems, K = (n + F - 1) / F;
  uint64_t total = al16(64 + 8 * K);
  for (uint64_t k = 0; k < K; k++) {
    const uint64_t Fk = std::min(F, n - k * F), raw = al16(Fk * w);
    switch (codec) {
      case CSWAP_CODEC_NONE: total += raw; break;
      case CSWAP_CODEC_ZVC: total += al16(4 * ((Fk + 31) / 32)) + raw; break;
      case CSWAP_CODEC_RLE: total += 16 + al16(4 * Fk) + raw; break;
      case CSWAP_CODEC_CSR: total += al16(4 * ((Fk + f.csr_row - 1) / f.csr_row + 1)) + al16(4 * Fk) + raw; break;
      case CSWAP_CODEC_LZ4: {
        const uint64_t bytes = Fk * w, B = f.lz4_block, nb = (bytes + B - 1) / B;
        uint64_t s = 0;
        for (uint64_t b = 0; b < nb; b++) {
          const uint64_t L = std::min(B, bytes - b * B);
          s += L + L / 255 + 16;
        }
        total += al16(4 * nb) + al16(s);
        break;
      }
      default: return 0;
    }
  }
  return total;
}

cswap_status cuda_status(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return CSWAP_OK;
  if (e == cudaErrorNotSupported) return fail(CSWAP_ERR_UNSUPPORTED, "%s: not implemented in this build", what);
  return fail(CSWAP_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

// ---- compress (device -> device or mapped) ---------------------------------------------------
cswap_status do_compress(Ctx* c, const void* in, uint64_t n, int dtype, int codec, const cswap_format& f,
                         uint8_t* out, uint64_t* out_size, cudaStream_t st) {
  const int w = width(dtype);
  const uint64_t F = f.frame_elems;
  const uint32_t K = uint32_t((n + F - 1) / F);
  if (n == 0) {
    c->launches++;
    return cuda_status(launch_header_only(out, codec, dtype, F, param_of(codec, f), out_size, st), "header");
  }
  switch (codec) {
    case CSWAP_CODEC_NONE:
      c->launches++;
      return cuda_status(launch_none_compress(in, n, w, F, dtype, out, out_size, st), "none_compress");
    case CSWAP_CODEC_ZVC: {
      uint64_t tiles = 0, aux = 0;
      zvc_compress_scratch(n, w, F, &tiles, &aux);
      Lease L(*c, st, tiles, aux);
      TRY(L.status);
      c->launches += 2;  // accumulator zero fill + persistent compress
      const uint32_t ep = L.epoch();
      return run_group(c, st, group_key(kGrpCompress, codec, dtype), [&](cudaStream_t gs) {
        return cuda_status(launch_zvc_compress(in, n, w, F, out, out_size, L.b->sc, ep, dtype, gs), "zvc_compress");
      });
    }
    case CSWAP_CODEC_RLE: {
      Lease L(*c, st, rle_tiles(n, w, F) + 2, uint64_t(K) + 2);
      TRY(L.status);
      c->launches += 4;
      const uint32_t ep = L.epoch();
      return run_group(c, st, group_key(kGrpCompress, codec, dtype), [&](cudaStream_t gs) {
        return cuda_status(launch_rle_compress(in, n, w, F, out, out_size, L.b->sc, ep, dtype, gs), "rle_compress");
      });
    }
    case CSWAP_CODEC_CSR: {
      Lease L(*c, st, rle_tiles(n, w, F) + 2, uint64_t(K) + 2);
      TRY(L.status);
      c->launches += 4;
      const uint32_t ep = L.epoch();
      return run_group(c, st, group_key(kGrpCompress, codec, dtype), [&](cudaStream_t gs) {
        return cuda_status(launch_csr_compress(in, n, w, F, f.csr_row, out, out_size, L.b->sc, ep, dtype, gs),
                           "csr_compress");
      });
    }
    case CSWAP_CODEC_LZ4: {
      const uint64_t blocks = lz4_scratch_bytes(n, w, F, f.lz4_block);
      uint8_t* slots = nullptr;
      CU(cudaMallocAsync(&slots, blocks, st));
      const uint64_t bidx = uint64_t(K) * ((F * w + f.lz4_block - 1) / f.lz4_block);  // block index k*bpf + b
      cswap_status s;
      {
        Lease L(*c, st, bidx + 2, uint64_t(K) + 2);
        TRY(L.status);
        c->launches += 3;
        s = run_group(c, st, group_key(kGrpCompress, codec, dtype), [&](cudaStream_t gs) {
          return cuda_status(launch_lz4_compress(in, n, w, F, f.lz4_block, out, out_size, slots, L.b->sc, dtype, gs),
                             "lz4_compress");
        });
      }
      CU(cudaFreeAsync(slots, st));
      return s;
    }
    default: return fail(CSWAP_ERR_INVALID, "unknown codec %d", codec);
  }
}

// ---- decompress frames [k0, k1) (prep must have run in the same lease) -----------------------
// `tmp`: caller-owned decode scratch (decompress_tmp_bytes), so the group allocates nothing and
// can be captured as a graph
cswap_status decompress_range(Ctx* c, Lease& L, const uint8_t* in, void* out, uint64_t n, int dtype, int codec,
                              const cswap_format& f, uint32_t k0, uint32_t k1, uint32_t* err, uint8_t* tmp,
                              cudaStream_t st) {
  const int w = width(dtype);
  const uint64_t F = f.frame_elems;
  switch (codec) {
    case CSWAP_CODEC_NONE: return CSWAP_OK;  // handled by the caller (raw copy)
    case CSWAP_CODEC_ZVC:
      c->launches += 3;  // count, scan, expand
      return cuda_status(launch_zvc_decompress(in, out, n, w, F, k0, k1, L.b->sc, 0, err, st), "zvc_decompress");
    case CSWAP_CODEC_RLE:
      c->launches += 4;  // chunk sums, chunk scan, runs, long-run fill
      return cuda_status(launch_rle_decompress(in, out, n, w, F, k0, k1, L.b->sc, 0, err, tmp, st), "rle_decompress");
    case CSWAP_CODEC_CSR:
      c->launches++;
      return cuda_status(launch_csr_decompress(in, out, n, w, F, f.csr_row, k0, k1, L.b->sc, err, st), "csr_decompress");
    case CSWAP_CODEC_LZ4:
      c->launches += 2;
      return cuda_status(launch_lz4_decompress(in, out, n, w, F, f.lz4_block, k0, k1, L.b->sc, err, st),
                         "lz4_decompress");
    default: return fail(CSWAP_ERR_INVALID, "unknown codec %d", codec);
  }
}

uint64_t decompress_tmp_bytes(int codec, uint64_t n, const cswap_format& f, uint32_t k0, uint32_t k1) {
  return codec == CSWAP_CODEC_RLE ? rle_decompress_tmp_bytes(n, f.frame_elems, k0, k1) : 0;
}

uint64_t decompress_tiles(uint64_t n, int w, const cswap_format& f) {
  const uint64_t F = f.frame_elems, K = (n + F - 1) / F;
  uint64_t t = zvc_tiles(n, w, F, 0, uint32_t(K), nullptr);
  t = std::max<uint64_t>(t, rle_tiles(n, w, F) + 2);
  t = std::max<uint64_t>(t, K * ((F * w + f.lz4_block - 1) / f.lz4_block));  // LZ4 block index k*bpf + b
  return t + 2;
}
uint64_t decompress_aux(uint64_t n, int w, const cswap_format& f) {
  const uint64_t F = f.frame_elems, K = (n + F - 1) / F;
  uint64_t nblk = 0;
  for (uint64_t k = 0; k < K; k++) nblk += (std::min(F, n - k * F) * w + f.lz4_block - 1) / f.lz4_block;
  return std::max<uint64_t>({K, nblk + K, rle_tiles(n, w, F)}) + 2;
}

cswap_status check_common(const void* p, const char* what) {
  if (!p) return fail(CSWAP_ERR_INVALID, "%s is NULL", what);
  if (reinterpret_cast<uintptr_t>(p) % 16) return fail(CSWAP_ERR_INVALID, "%s must be 16-byte aligned", what);
  return CSWAP_OK;
}

}  // namespace

// =============================================================================================
// swap handle
// =============================================================================================
struct cswap_handle {
  Ctx* ctx = nullptr;
  uint8_t* host = nullptr;  // container (pinned pool)
  uint64_t bytes = 0;       // container bytes
  uint64_t n = 0;
  int dtype = 0, codec = 0;
  cswap_format fmt{};
  cswap_decision dec{};
  cudaEvent_t ev_out = nullptr, ev_in = nullptr;
  bool in_issued = false;
  uint8_t* slots = nullptr;  // pinned small slots: [0..8) size, [8..12) err
  uint64_t* size_slot() { return reinterpret_cast<uint64_t*>(slots); }
  uint32_t* err_slot() { return reinterpret_cast<uint32_t*>(slots + 64); }
};

// =============================================================================================
// C ABI
// =============================================================================================
extern "C" {

const char* cswap_status_string(cswap_status s) {
  switch (s) {
    case CSWAP_OK: return "ok";
    case CSWAP_ERR_INVALID: return "invalid argument";
    case CSWAP_ERR_CUDA: return "CUDA error";
    case CSWAP_ERR_NOMEM: return "out of memory";
    case CSWAP_ERR_CAPACITY: return "output capacity too small";
    case CSWAP_ERR_CORRUPT: return "corrupt container";
    case CSWAP_ERR_UNSUPPORTED: return "unsupported";
    case CSWAP_ERR_NOT_READY: return "not initialised";
  }
  return "unknown status";
}

const char* cswap_last_error(void) { return g_err.c_str(); }

uint64_t cswap_kernel_launches(void) { return g_ctx ? g_ctx->launches.load() : 0; }

void cswap_graph_stats(uint64_t* launches, uint64_t* instantiations) {
  if (launches) *launches = g_ctx ? g_ctx->graph_launches.load() : 0;
  if (instantiations) *instantiations = g_ctx ? g_ctx->graph_instantiations.load() : 0;
}

cswap_status cswap_init(int device) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g_ctx) {
    if (g_ctx->device == device) return CSWAP_OK;
    return fail(CSWAP_ERR_INVALID, "already initialised on device %d", g_ctx->device);
  }
  CU(cudaSetDevice(device));
  Ctx* c = new Ctx();
  c->device = device;
  c->gen = ++g_gen;
  CU(cudaDeviceGetAttribute(&c->sms, cudaDevAttrMultiProcessorCount, device));
  CU(cudaStreamCreateWithFlags(&c->s_d2h, cudaStreamNonBlocking));
  CU(cudaStreamCreateWithFlags(&c->s_h2d, cudaStreamNonBlocking));
  for (auto& b : c->blocks) {
    CU(cudaEventCreateWithFlags(&b.ev, cudaEventDisableTiming));
    TRY(ensure_block(b, 1 << 16, 1 << 12));
  }
  cudaMemPool_t pool;
  CU(cudaDeviceGetDefaultMemPool(&pool, device));
  uint64_t thr = UINT64_MAX;
  CU(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
  CU(cudaMalloc(&c->dev_err, 64));
  CU(cudaMemset(c->dev_err, 0, 64));
  if (const char* e = getenv("CSWAP_PINNED_CHUNK_MB")) c->pinned.chunk_bytes = uint64_t(atoll(e)) << 20;
  c->calib = builtin_calib();
  c->fmt = cswap_format{uint64_t(1) << 22, 1024, 65536};
  g_ctx = c;
  return CSWAP_OK;
}

cswap_status cswap_shutdown(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g_ctx) return CSWAP_OK;
  Ctx* c = g_ctx;
  cudaDeviceSynchronize();
  for (auto& b : c->blocks) {
    cudaFree(b.sc.status);
    cudaFree(b.sc.tickets);
    cudaFree(b.sc.aux);
    cudaFree(b.sc.aux2);
    cudaFree(b.sc.err);
    cudaFree(b.sc.tbuf);
    cudaFree(b.sc.tbuf2);
    cudaFree(b.sc.aux3);
    cudaEventDestroy(b.ev);
  }
  cudaFree(c->dev_err);
  cudaStreamDestroy(c->s_d2h);
  cudaStreamDestroy(c->s_h2d);
  c->pinned.destroy();
  delete c;
  g_ctx = nullptr;
  return CSWAP_OK;
}

cswap_status cswap_set_calibration(const cswap_calib* cal) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  if (!cal || cal->bw_d2h <= 0 || cal->bw_h2d <= 0 || cal->frame_elems == 0 || cal->csr_row == 0 || cal->lz4_block == 0)
    return fail(CSWAP_ERR_INVALID, "bad calibration");
  std::lock_guard<std::mutex> lk(c->cfg_m);
  c->calib = *cal;
  return CSWAP_OK;
}

cswap_status cswap_get_calibration(cswap_calib* out) {
  if (!out) return fail(CSWAP_ERR_INVALID, "out is NULL");
  if (!g_ctx) {
    *out = builtin_calib();
    return CSWAP_OK;
  }
  std::lock_guard<std::mutex> lk(g_ctx->cfg_m);
  *out = g_ctx->calib;
  return CSWAP_OK;
}

cswap_status cswap_set_format(const cswap_format* f) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  if (!f) return fail(CSWAP_ERR_INVALID, "fmt is NULL");
  TRY(check_fmt(*f));
  std::lock_guard<std::mutex> lk(c->cfg_m);
  c->fmt = *f;
  c->calib.frame_elems = f->frame_elems;
  c->calib.csr_row = f->csr_row;
  c->calib.lz4_block = f->lz4_block;
  return CSWAP_OK;
}

cswap_status cswap_set_zvc_launch(uint32_t grid, int32_t variant) {
  if (!zvc_set_launch(grid, variant)) return fail(CSWAP_ERR_INVALID, "variant %d outside -1..3", int(variant));
  return CSWAP_OK;
}

cswap_status cswap_get_format(cswap_format* out) {
  if (!out) return fail(CSWAP_ERR_INVALID, "out is NULL");
  *out = g_ctx ? g_ctx->fmt : cswap_format{uint64_t(1) << 22, 1024, 65536};
  return CSWAP_OK;
}

uint64_t cswap_max_compressed_size(uint64_t n, cswap_dtype dtype, cswap_codec codec, const cswap_format* fmt) {
  const int w = width(dtype);
  cswap_format f = fmt ? *fmt : (g_ctx ? g_ctx->fmt : cswap_format{uint64_t(1) << 22, 1024, 65536});
  if (!w || check_fmt(f) != CSWAP_OK) return 0;
  return max_size(n, w, codec, f);
}

cswap_status cswap_compress(const void* d_in, uint64_t n, cswap_dtype dtype, cswap_codec codec,
                            const cswap_format* fmt, void* out, uint64_t out_cap, uint64_t* out_size, void* stream) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  const int w = width(dtype);
  if (!w) return fail(CSWAP_ERR_INVALID, "bad dtype %d", int(dtype));
  if (codec > CSWAP_CODEC_LZ4) return fail(CSWAP_ERR_INVALID, "codec must be NONE/ZVC/RLE/CSR/LZ4");
  if (n) TRY(check_common(d_in, "d_in"));
  TRY(check_common(out, "out"));
  if (!out_size) return fail(CSWAP_ERR_INVALID, "out_size is NULL");
  const cswap_format f = resolve_fmt(c, fmt);
  TRY(check_fmt(f));
  if (out_cap < max_size(n, w, codec, f))
    return fail(CSWAP_ERR_CAPACITY, "out_cap %llu < %llu", (unsigned long long)out_cap,
                (unsigned long long)max_size(n, w, codec, f));
  return do_compress(c, d_in, n, dtype, codec, f, static_cast<uint8_t*>(out), out_size,
                     static_cast<cudaStream_t>(stream));
}

cswap_status cswap_decompress(const void* in, uint64_t in_size, void* d_out, uint64_t n, cswap_dtype dtype,
                              cswap_codec codec, const cswap_format* fmt, uint32_t* err, void* stream) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  const int w = width(dtype);
  if (!w) return fail(CSWAP_ERR_INVALID, "bad dtype %d", int(dtype));
  if (codec > CSWAP_CODEC_LZ4) return fail(CSWAP_ERR_INVALID, "codec must be NONE/ZVC/RLE/CSR/LZ4");
  TRY(check_common(in, "in"));
  if (n) TRY(check_common(d_out, "d_out"));
  if (in_size < 64) return fail(CSWAP_ERR_CORRUPT, "in_size < 64");
  const cswap_format f = resolve_fmt(c, fmt);
  TRY(check_fmt(f));
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  uint32_t* user_err = err ? err : c->dev_err;
  const uint64_t F = f.frame_elems;
  const uint32_t K = uint32_t((n + F - 1) / F);
  Lease L(*c, st, decompress_tiles(n, w, f), decompress_aux(n, w, f));
  TRY(L.status);
  // kernels flag errors in the lease's device word (never in host-mapped memory: every CTA
  // reads it); the word is merged into the caller's at the end
  uint32_t* e = L.b->sc.err;
  const uint8_t* inb = static_cast<const uint8_t*>(in);
  uint8_t* tmp = nullptr;
  const uint64_t tmp_bytes = n ? decompress_tmp_bytes(codec, n, f, 0, K) : 0;
  if (tmp_bytes) CU(cudaMallocAsync(&tmp, tmp_bytes, st));
  c->launches += 2;  // prep, err merge (+ the codec's kernels)
  cswap_status s = run_group(c, st, group_key(kGrpDecompress, codec, dtype), [&](cudaStream_t gs) {
    TRY(cuda_status(launch_prep(inb, in_size, codec, dtype, n, F, param_of(codec, f), L.b->sc, e, true, gs), "prep"));
    if (n != 0) {
      if (codec == CSWAP_CODEC_NONE) {
        c->launches++;
        TRY(cuda_status(launch_none_decompress(inb, d_out, n, w, F, L.b->sc, e, gs), "none_decompress"));
      } else {
        TRY(decompress_range(c, L, inb, d_out, n, dtype, codec, f, 0, K, e, tmp, gs));
      }
    }
    return cuda_status(launch_err_merge(e, user_err, gs), "err_merge");
  });
  if (tmp) cudaFreeAsync(tmp, st);
  return s;
}

cswap_status cswap_check_device_error(void* stream) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  CU(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
  uint32_t v = 0;
  CU(cudaMemcpy(&v, c->dev_err, 4, cudaMemcpyDeviceToHost));
  if (v) {
    CU(cudaMemset(c->dev_err, 0, 4));
    return fail(CSWAP_ERR_CORRUPT, "device-side validation failed (code %u)", v);
  }
  return CSWAP_OK;
}

// ---- probe / select --------------------------------------------------------------------------
static cswap_status probe_impl(Ctx* c, const void* d_in, uint64_t n, int dtype, cswap_probe_result* out,
                               cudaStream_t st) {
  const int w = width(dtype);
  std::memset(out, 0, sizeof(*out));
  if (n == 0) return CSWAP_OK;
  uint8_t* slot = c->pinned.alloc(256);
  if (!slot) return fail(CSWAP_ERR_NOMEM, "pinned alloc failed");
  uint64_t* counts = reinterpret_cast<uint64_t*>(slot);
  cudaEvent_t ev;
  cswap_status s = CSWAP_OK;
  // spin-wait event: a blocking-sync event sleeps in the OS and wakes ~100 us late
  if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess) {
    c->pinned.free(slot);
    return fail(CSWAP_ERR_CUDA, "event create failed");
  }
  {
    Lease L(*c, st, 1024, 1024);
    s = L.status;
    if (s == CSWAP_OK) {
      Timer tm(c, st);
      c->launches++;
      s = cuda_status(launch_probe(d_in, n, w, counts, L.b->sc, L.epoch(), st), "probe");
      tm.commit(0, 2, std::min<uint64_t>(n, 262144) * w, 0);
    }
    if (s == CSWAP_OK && cudaEventRecord(ev, st) != cudaSuccess) s = fail(CSWAP_ERR_CUDA, "event record");
  }
  if (s == CSWAP_OK && cudaEventSynchronize(ev) != cudaSuccess) s = fail(CSWAP_ERR_CUDA, "probe sync failed");
  if (s == CSWAP_OK) {
    const bool single = n <= 262144;
    out->zeros = counts[0];
    out->zero_runs = counts[1];
    out->boundaries = counts[2];
    out->samples = single ? n : 262144;
    out->pairs = out->samples - (single ? 1 : 1024);
  }
  cudaEventDestroy(ev);
  c->pinned.free(slot);
  return s;
}

cswap_status cswap_probe(const void* d_in, uint64_t n, cswap_dtype dtype, cswap_probe_result* out, void* stream) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  if (!width(dtype)) return fail(CSWAP_ERR_INVALID, "bad dtype");
  if (!out) return fail(CSWAP_ERR_INVALID, "out is NULL");
  if (n && !d_in) return fail(CSWAP_ERR_INVALID, "d_in is NULL");
  return probe_impl(c, d_in, n, dtype, out, static_cast<cudaStream_t>(stream));
}

cswap_status cswap_select_from_probe(uint64_t n, cswap_dtype dtype, const cswap_probe_result* probe, double hidden_f,
                                     double hidden_b, const cswap_calib* calib, cswap_decision* out) {
  const int w = width(dtype);
  if (!w || !probe || !out) return fail(CSWAP_ERR_INVALID, "bad arguments");
  cswap_calib cal;
  if (calib) cal = *calib;
  else cswap_get_calibration(&cal);
  if (cal.bw_d2h <= 0 || cal.bw_h2d <= 0 || cal.frame_elems == 0 || cal.csr_row == 0 || cal.lz4_block == 0)
    return fail(CSWAP_ERR_INVALID, "bad calibration");
  decide(n, w, *probe, hidden_f, hidden_b, cal, out);
  return CSWAP_OK;
}

cswap_status cswap_select(const void* d_in, uint64_t n, cswap_dtype dtype, double hidden_f, double hidden_b,
                          void* stream, cswap_decision* out) {
  cswap_probe_result p;
  TRY(cswap_probe(d_in, n, dtype, &p, stream));
  return cswap_select_from_probe(n, dtype, &p, hidden_f, hidden_b, nullptr, out);
}

// ---- swap pipeline ---------------------------------------------------------------------------
cswap_status cswap_swap_out(const void* d_in, uint64_t n, cswap_dtype dtype, cswap_codec codec, double hidden_f,
                            double hidden_b, void* stream, cswap_handle** out) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  const int w = width(dtype);
  if (!w || !out) return fail(CSWAP_ERR_INVALID, "bad arguments");
  if (n) TRY(check_common(d_in, "d_in"));
  if (codec > CSWAP_CODEC_LZ4 && codec != CSWAP_CODEC_AUTO) return fail(CSWAP_ERR_INVALID, "bad codec");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const cswap_format f = resolve_fmt(c, nullptr);
  auto* h = new cswap_handle();
  h->ctx = c;
  h->n = n;
  h->dtype = dtype;
  h->fmt = f;
  h->slots = c->pinned.alloc(256);
  if (!h->slots) {
    delete h;
    return fail(CSWAP_ERR_NOMEM, "pinned alloc failed");
  }
  auto bail = [&](cswap_status s) {
    cswap_handle_free(h);
    return s;
  };
  if (cudaEventCreateWithFlags(&h->ev_out, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&h->ev_in, cudaEventDisableTiming) != cudaSuccess)
    return bail(fail(CSWAP_ERR_CUDA, "event create failed"));
  int use = codec;
  if (codec == CSWAP_CODEC_AUTO) {
    cswap_probe_result p;
    cswap_status s = probe_impl(c, d_in, n, dtype, &p, st);
    if (s != CSWAP_OK) return bail(s);
    cswap_calib cal;
    cswap_get_calibration(&cal);
    decide(n, w, p, hidden_f, hidden_b, cal, &h->dec);
    use = h->dec.codec;
  } else {
    h->dec.codec = codec;
  }
  h->codec = use;
  const uint64_t F = f.frame_elems;
  const uint32_t K = uint32_t((n + F - 1) / F);
  cudaEvent_t ready;
  if (cudaEventCreateWithFlags(&ready, cudaEventDisableTiming) != cudaSuccess)
    return bail(fail(CSWAP_ERR_CUDA, "event create failed"));
  if (use == CSWAP_CODEC_NONE) {
    // raw offload: host writes header + frame table, the copy engine moves the frames
    const uint64_t cap = max_size(n, w, CSWAP_CODEC_NONE, f);
    h->host = c->pinned.alloc(cap);
    if (!h->host) return bail(fail(CSWAP_ERR_NOMEM, "pinned alloc of %llu B failed", (unsigned long long)cap));
    std::memset(h->host, 0, al16(64 + 8ull * K));
    const uint64_t tail = al16(64 + 8ull * K) + uint64_t(w) * n;
    std::memset(h->host + tail, 0, cap - tail);
    uint64_t total = al16(64 + 8ull * K);
    for (uint32_t k = 0; k < K; k++) {
      const uint64_t fb = al16(uint64_t(w) * std::min<uint64_t>(F, n - uint64_t(k) * F));
      std::memcpy(h->host + 64 + 8ull * k, &fb, 8);
      total += fb;
    }
    std::memcpy(h->host, "CSWP", 4);
    const uint16_t ver = 1;
    std::memcpy(h->host + 4, &ver, 2);
    h->host[6] = 0;
    h->host[7] = uint8_t(dtype);
    std::memcpy(h->host + 8, &n, 8);
    std::memcpy(h->host + 16, &F, 8);
    std::memcpy(h->host + 24, &K, 4);
    std::memcpy(h->host + 32, &total, 8);
    h->bytes = total;
    if (n) {
      if (cudaEventRecord(ready, st) != cudaSuccess || cudaStreamWaitEvent(c->s_d2h, ready, 0) != cudaSuccess ||
          cudaMemcpyAsync(h->host + al16(64 + 8ull * K), d_in, uint64_t(w) * n, cudaMemcpyDeviceToHost, c->s_d2h) !=
              cudaSuccess) {
        cudaEventDestroy(ready);
        return bail(fail(CSWAP_ERR_CUDA, "raw offload failed"));
      }
    }
    cudaEventRecord(h->ev_out, c->s_d2h);
    cudaEventDestroy(ready);
    *out = h;
    return CSWAP_OK;
  }
  // compressed offload: compress into stream-ordered device staging, read the size, D2H
  const uint64_t cap = max_size(n, w, use, f);
  uint8_t* staging = nullptr;
  cswap_status s = CSWAP_OK;
  if (cudaMallocAsync(&staging, cap, st) != cudaSuccess) {
    cudaEventDestroy(ready);
    return bail(fail(CSWAP_ERR_NOMEM, "device staging of %llu B failed", (unsigned long long)cap));
  }
  Timer tm(c, st);
  s = do_compress(c, d_in, n, dtype, use, f, staging, h->size_slot(), st);
  tm.stop();
  if (s == CSWAP_OK && cudaEventRecord(ready, st) != cudaSuccess) s = fail(CSWAP_ERR_CUDA, "event record");
  if (s == CSWAP_OK && cudaEventSynchronize(ready) != cudaSuccess) s = fail(CSWAP_ERR_CUDA, "compress failed");
  if (s == CSWAP_OK) {
    h->bytes = *h->size_slot();
    tm.commit(use, 0, n * uint64_t(w), h->bytes);
    h->host = c->pinned.alloc(h->bytes);
    if (!h->host) s = fail(CSWAP_ERR_NOMEM, "pinned alloc of %llu B failed", (unsigned long long)h->bytes);
  }
  if (s == CSWAP_OK && (cudaStreamWaitEvent(c->s_d2h, ready, 0) != cudaSuccess ||
                        cudaMemcpyAsync(h->host, staging, h->bytes, cudaMemcpyDeviceToHost, c->s_d2h) != cudaSuccess))
    s = fail(CSWAP_ERR_CUDA, "offload copy failed");
  cudaFreeAsync(staging, s == CSWAP_OK ? c->s_d2h : st);
  cudaEventRecord(h->ev_out, c->s_d2h);
  cudaEventDestroy(ready);
  if (s != CSWAP_OK) return bail(s);
  *out = h;
  return CSWAP_OK;
}

cswap_status cswap_swap_in(cswap_handle* h, void* d_out, void* stream) {
  if (!h) return fail(CSWAP_ERR_INVALID, "handle is NULL");
  Ctx* c = h->ctx;
  const int w = width(h->dtype);
  if (h->n) TRY(check_common(d_out, "d_out"));
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const cswap_format& f = h->fmt;
  const uint64_t F = f.frame_elems, n = h->n;
  const uint32_t K = uint32_t((n + F - 1) / F);
  CU(cudaEventSynchronize(h->ev_out));  // the host container (header, frame table) is complete
  h->in_issued = true;
  *h->err_slot() = 0;
  if (n == 0) return cudaEventRecord(h->ev_in, st) == cudaSuccess ? CSWAP_OK : fail(CSWAP_ERR_CUDA, "record");
  cudaEvent_t ready;
  CU(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming));
  CU(cudaEventRecord(ready, st));
  CU(cudaStreamWaitEvent(c->s_h2d, ready, 0));
  if (h->codec == CSWAP_CODEC_NONE) {
    CU(cudaMemcpyAsync(d_out, h->host + al16(64 + 8ull * K), uint64_t(w) * n, cudaMemcpyHostToDevice, c->s_h2d));
    CU(cudaEventRecord(h->ev_in, c->s_h2d));
    CU(cudaStreamWaitEvent(st, h->ev_in, 0));
    cudaEventDestroy(ready);
    return CSWAP_OK;
  }
  // pipelined prefetch: groups of frames of ~64 MiB raw; H2D(g+1) overlaps decompress(g)
  const uint64_t* fb = reinterpret_cast<const uint64_t*>(h->host + 64);
  uint8_t* staging = nullptr;
  CU(cudaMallocAsync(&staging, h->bytes, c->s_h2d));
  const uint64_t group_raw = uint64_t(64) << 20;
  const uint32_t fpg = uint32_t(std::max<uint64_t>(1, group_raw / (F * w)));
  std::vector<cudaEvent_t> evs;
  cswap_status s = CSWAP_OK;
  {
    Lease L(*c, st, decompress_tiles(n, w, f), decompress_aux(n, w, f));
    s = L.status;
    uint32_t* e_dev = L.b->sc.err;  // device word; merged into the handle's pinned slot at the end
    uint64_t off = 0;
    for (uint32_t k0 = 0; k0 < K && s == CSWAP_OK; k0 += fpg) {
      const uint32_t k1 = std::min(K, k0 + fpg);
      uint64_t end = al16(64 + 8ull * K);
      for (uint32_t k = 0; k < k1; k++) end += fb[k];
      if (k1 == K) end = h->bytes;
      cudaEvent_t e;
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) {
        s = fail(CSWAP_ERR_CUDA, "event create");
        break;
      }
      evs.push_back(e);
      if (cudaMemcpyAsync(staging + off, h->host + off, end - off, cudaMemcpyHostToDevice, c->s_h2d) != cudaSuccess ||
          cudaEventRecord(e, c->s_h2d) != cudaSuccess || cudaStreamWaitEvent(st, e, 0) != cudaSuccess) {
        s = fail(CSWAP_ERR_CUDA, "prefetch copy failed");
        break;
      }
      uint8_t* tmp = nullptr;
      const uint64_t tmp_bytes = decompress_tmp_bytes(h->codec, n, f, k0, k1);
      if (tmp_bytes && cudaMallocAsync(&tmp, tmp_bytes, st) != cudaSuccess) {
        s = fail(CSWAP_ERR_NOMEM, "decode scratch");
        break;
      }
      Timer tm(c, st);
      const bool first = k0 == 0, last = k1 == K;
      c->launches += (first ? 1 : 0) + (last ? 1 : 0);
      s = run_group(c, st, group_key(first ? kGrpSwapInFirst : kGrpSwapIn, h->codec, h->dtype) | (last ? 1u << 20 : 0),
                    [&](cudaStream_t gs) {
                      if (first)
                        TRY(cuda_status(launch_prep(staging, h->bytes, h->codec, h->dtype, n, F,
                                                    param_of(h->codec, f), L.b->sc, e_dev, true, gs),
                                        "prep"));
                      TRY(decompress_range(c, L, staging, d_out, n, h->dtype, h->codec, f, k0, k1, e_dev, tmp, gs));
                      // the last group folds the device error word into the handle's pinned slot
                      if (last) TRY(cuda_status(launch_err_merge(e_dev, h->err_slot(), gs), "err_merge"));
                      return CSWAP_OK;
                    });
      if (tmp) cudaFreeAsync(tmp, st);
      const uint64_t raw = (std::min<uint64_t>(n, uint64_t(k1) * F) - uint64_t(k0) * F) * w;
      tm.commit(h->codec, 1, raw, end - off);
      off = end;
    }
  }
  cudaFreeAsync(staging, st);
  cudaEventRecord(h->ev_in, st);
  for (auto e : evs) cudaEventDestroy(e);
  cudaEventDestroy(ready);
  return s;
}

cswap_status cswap_handle_wait(cswap_handle* h) {
  if (!h) return fail(CSWAP_ERR_INVALID, "handle is NULL");
  CU(cudaEventSynchronize(h->ev_out));
  if (h->in_issued) {
    CU(cudaEventSynchronize(h->ev_in));
    if (*h->err_slot()) return fail(CSWAP_ERR_CORRUPT, "swap-in validation failed");
  }
  return CSWAP_OK;
}

cswap_status cswap_handle_record_out(cswap_handle* h, void* stream) {
  if (!h) return fail(CSWAP_ERR_INVALID, "handle is NULL");
  CU(cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), h->ev_out, 0));
  return CSWAP_OK;
}

cswap_status cswap_handle_query(const cswap_handle* h, cswap_codec* codec, uint64_t* container_bytes,
                                const void** host_container, cswap_decision* decision) {
  if (!h) return fail(CSWAP_ERR_INVALID, "handle is NULL");
  if (codec) *codec = cswap_codec(h->codec);
  if (container_bytes) *container_bytes = h->bytes;
  if (host_container) *host_container = h->host;
  if (decision) *decision = h->dec;
  return CSWAP_OK;
}

void cswap_handle_free(cswap_handle* h) {
  if (!h) return;
  if (h->ev_out) cudaEventSynchronize(h->ev_out);
  if (h->ev_in && h->in_issued) cudaEventSynchronize(h->ev_in);
  if (h->ev_out) cudaEventDestroy(h->ev_out);
  if (h->ev_in) cudaEventDestroy(h->ev_in);
  h->ctx->pinned.free(h->host);
  h->ctx->pinned.free(h->slots);
  delete h;
}

cswap_status cswap_fit_time_model(const double* S, const double* s, const double* t, uint64_t m, double* beta_out) {
  if (!S || !s || !t || !beta_out) return fail(CSWAP_ERR_INVALID, "NULL argument");
  if (!fit3(S, s, t, m, beta_out)) return fail(CSWAP_ERR_INVALID, "singular or too few samples");
  return CSWAP_OK;
}

cswap_status cswap_fit_linear(const double* X, const double* y, uint64_t m, uint32_t p, double* beta_out) {
  if (!X || !y || !beta_out) return fail(CSWAP_ERR_INVALID, "NULL argument");
  if (!fit_general(X, y, m, p, beta_out)) return fail(CSWAP_ERR_INVALID, "singular, p > 8 or m < p");
  return CSWAP_OK;
}

cswap_status cswap_set_kernel_timing(int enable) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  c->timing.store(enable != 0);
  return CSWAP_OK;
}

uint64_t cswap_collect_kernel_timing(cswap_kernel_record* out, uint64_t cap) {
  if (!g_ctx) return 0;
  Ctx* c = g_ctx;
  std::vector<Ctx::Pend> p;
  {
    std::lock_guard<std::mutex> lk(c->tm_m);
    p.swap(c->pend);
  }
  uint64_t k = 0;
  for (auto& e : p) {
    float ms = 0;
    cudaEventSynchronize(e.b);
    cudaEventElapsedTime(&ms, e.a, e.b);
    e.r.ms = ms;
    if (e.stamps) {  // written by the group's stamp kernels, complete once e.b is
      const volatile uint64_t* t = e.stamps;
      e.r.device_ms = (t[0] && t[1] > t[0]) ? double(t[1] - t[0]) * 1e-6 : 0.0;
      c->pinned.free(reinterpret_cast<uint8_t*>(e.stamps));
    }
    if (out && k < cap) out[k] = e.r;
    k++;
    cudaEventDestroy(e.a);
    cudaEventDestroy(e.b);
  }
  return std::min(k, cap);
}

cswap_status cswap_fit_link(const double* bytes, const double* t, uint64_t m, double* alpha_out, double* bw_out) {
  if (!bytes || !t || !alpha_out || !bw_out) return fail(CSWAP_ERR_INVALID, "NULL argument");
  if (!fit_link(bytes, t, m, alpha_out, bw_out)) return fail(CSWAP_ERR_INVALID, "degenerate link samples");
  return CSWAP_OK;
}

}  // extern "C"
