// api.cu — the C ABI of include/cswap.h: runtime (streams, scratch, pools, handles, the swap-out
// executor thread), codec dispatch, probe + selector, and the swap-out / swap-in pipelines.
//
// Swapping executor (PAPER.md:120 §IV-A; :228 §V): compress -> offload to pinned host memory on
// an asynchronous copy stream; prefetch -> decompress.  Memory pools replace cudaMalloc /
// cudaMallocHost on the path: device staging comes from a private stream-ordered
// pool, host containers from a pinned-chunk allocator.  Both directions are pipelined per frame
// (R7): swap-out hands each frame to the copy engine as soon as the compress kernel
// publishes it (a library thread issues the D2H copies; the caller never blocks), swap-in's H2D
// of frame k+1 overlaps the decompression of frame k.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstdarg>
#include <deque>
#include <thread>
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

  uint8_t* take(uint64_t bytes) {  // first fit; caller holds m
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
    return nullptr;
  }
  uint8_t* alloc(uint64_t bytes) {
    bytes = round(bytes);
    uint64_t pinned_total = 0;
    {
      std::lock_guard<std::mutex> lk(m);
      if (uint8_t* p = take(bytes)) return p;
      for (auto& ch : chunks) pinned_total += ch.size;
    }
    // new chunks grow geometrically (at least half of what is pinned already): pinning host
    // memory costs milliseconds per GiB, so a workload reaches its steady footprint after a few
    // allocations instead of pinning a chunk on every swap once the pool is fragmented.  The
    // pinning runs outside the lock, so other threads' allocations are not held behind it.
    const uint64_t sz = std::max({bytes, chunk_bytes, (pinned_total / 2 + 255) / 256 * 256});
    void* p = nullptr;
    if (cudaHostAlloc(&p, sz, cudaHostAllocPortable | cudaHostAllocMapped) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    std::lock_guard<std::mutex> lk(m);
    chunks.push_back(Chunk{static_cast<uint8_t*>(p), sz, {}});
    chunks.back().free[0] = sz;
    return take(bytes);
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
  // unpin chunks that hold no live allocation (indices in `live` are renumbered)
  uint64_t release_empty() {
    std::lock_guard<std::mutex> lk(m);
    std::vector<bool> used(chunks.size(), false);
    for (auto& kv : live) used[kv.second.first] = true;
    std::vector<size_t> remap(chunks.size(), SIZE_MAX);
    std::vector<Chunk> keep;
    uint64_t freed = 0;
    for (size_t c = 0; c < chunks.size(); c++) {
      if (used[c]) {
        remap[c] = keep.size();
        keep.push_back(std::move(chunks[c]));
      } else {
        cudaFreeHost(chunks[c].base);
        freed += chunks[c].size;
      }
    }
    for (auto& kv : live) kv.second.first = remap[kv.second.first];
    chunks = std::move(keep);
    return freed;
  }
};

// ---------------------------------------------------------------------------------------------
// scratch blocks (tile status words, tickets, per-frame arrays) leased per operation
// ---------------------------------------------------------------------------------------------
struct Block {
  Scratch sc{};
  cudaEvent_t ev = nullptr;
  uint32_t epoch = 0;
  std::mutex m;
};

constexpr int kBlocks = 4;

struct OutJob;

struct Ctx {
  int device = -1;
  int sms = 0;
  Block blocks[kBlocks];
  std::atomic<uint32_t> rr{0};
  // D2H copy stream; two H2D copy streams that swap-in frames alternate between (an event record
  // on a copy stream stalls that stream ~25-35 us while PCIe is busy, tools/event_probe.cu: the
  // other stream's copy keeps the link busy meanwhile)
  cudaStream_t s_d2h = nullptr, s_h2d = nullptr, s_h2d2 = nullptr;
  // progress stream: copies a swap-out's device-side progress words to the host once its codec
  // group is done (the codec kernels then store no host memory: a kernel that does completes only
  // after its store drained behind the D2H queue, ~15-25 us of the caller's stream, §7.3)
  cudaStream_t s_prog = nullptr;
  cudaMemPool_t pool = nullptr;  // private stream-ordered pool (staging, LZ4 slots, decode scratch)
  uint64_t* dev_sink = nullptr;  // device word for container sizes nobody reads
  // kernel-timing stamps (cswap_set_kernel_timing): a ring of 3-word slots in DEVICE memory.  A
  // kernel that writes host-mapped memory while a copy streams over PCIe cannot complete until
  // its write drains behind the copy's (~20-25 us, tools/event_gap_probe.cu), so stamps there
  // would inflate the very duration they measure
  static constexpr uint32_t kStampSlots = 1u << 14, kStampWords = 5;
  uint64_t* dev_stamps = nullptr;
  std::atomic<uint32_t> stamp_next{0};
  // swap target (cswap_set_swap_target): -1 = pinned host; else a device whose memory holds the
  // containers (tpool: a pool located on that device, accessible from this one)
  int target = -1;
  cudaMemPool_t tpool = nullptr;
  // swap-out executor: one library thread turns published frames into D2H copies, FIFO
  std::thread exec;
  std::mutex qm;
  std::condition_variable qcv;
  std::deque<OutJob*> q;
  bool stop = false;

  std::mutex cfg_m;
  cswap_calib calib{};
  cswap_format fmt{};
  PinnedPool pinned;  // host containers
  PinnedPool small;   // progress words, probe counts, timer stamps, handle slots (never wait on a container's pinning)
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
    uint64_t* stamps;  // device slot: 2 x u64 %globaltimer, the container size, kernel clock[2]; or null
    bool stamped, self_clocked;  // which words of the slot this group wrote
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
  // device slot — [0], [1]: filled by stamp kernels first / last in the group (run_group; the first
  // also clears [1] and [2]); [2]: a swap-out's compress writes its container size here (all
  // three are read at collection time)
  uint64_t* stamps = nullptr;
  bool stamped = false;  // a group's stamp kernels were enqueued (else words 0, 1 are stale)
  // the group's kernel clocks itself (words 3, 4) and writes the container size (word 2): no stamp
  // kernels, whose boundaries cost ~12 us each while a copy streams
  bool self_clocked = false;
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
    c->pend.push_back(Ctx::Pend{a, b, cswap_kernel_record{codec, dir, raw, comp, 0.0, 0.0, 0.0},
                                (stamped || self_clocked) ? stamps : nullptr, stamped, self_clocked});
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
    if (c->dev_stamps)
      stamps = c->dev_stamps + uint64_t(Ctx::kStampWords) * (c->stamp_next.fetch_add(1) % Ctx::kStampSlots);
  }
}
Timer::~Timer() {
  if (t_pending == this) t_pending = nullptr;
  if (a) cudaEventDestroy(a);
  if (b) cudaEventDestroy(b);
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
  uint64_t* stamps = pending && !pending->self_clocked ? pending->stamps : nullptr;
  // timed groups: stamp kernels first and last (device duration of the group)
  auto body = [&](cudaStream_t gs) -> cswap_status {
    if (stamps) {
      c->launches++;
      TRY(cuda_status(launch_stamp(stamps, gs, true), "stamp"));
      pending->stamped = true;
    }
    TRY(fn(gs));
    if (stamps) {
      c->launches++;
      TRY(cuda_status(launch_stamp(stamps + 1, gs, false), "stamp"));
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
    cudaFree(b.sc.zacc);
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
  CU(cudaMalloc(&b.sc.zacc, aux * 8));
  CU(cudaMemset(b.sc.status, 0, tiles * 8));
  // epoch-tagged words are also polled in aux (frame starts): a fresh block restarts at epoch 0,
  // so memory recycled from an earlier block could hold words tagged with a live epoch; zero
  // every scratch array once (compute-sanitizer initcheck flagged the first reads of aux)
  CU(cudaMemset(b.sc.aux, 0, aux * 8));
  CU(cudaMemset(b.sc.aux2, 0, aux * 8));
  CU(cudaMemset(b.sc.aux3, 0, aux * 8));
  CU(cudaMemset(b.sc.zacc, 0, aux * 8));
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
// prog (swap-out only): host-mapped progress words, see Scratch::prog.  ZVC publishes each frame
// from inside its persistent kernel; the multi-pass codecs publish every frame once their last
// kernel has run (a publish kernel at the end of the same launch group).
cswap_status do_compress(Ctx* c, const void* in, uint64_t n, int dtype, int codec, const cswap_format& f,
                         uint8_t* out, uint64_t* out_size, cudaStream_t st, uint64_t* prog = nullptr,
                         bool frame_publish = false) {
  const int w = width(dtype);
  const uint64_t F = f.frame_elems;
  const uint32_t K = uint32_t((n + F - 1) / F);
  auto publish = [&](cudaStream_t gs) -> cswap_status {
    if (!prog) return CSWAP_OK;
    c->launches++;
    return cuda_status(launch_publish_frames(out, K, prog, gs), "publish_frames");
  };
  auto with_prog = [&](const Scratch& sc, uint32_t mode) {
    Scratch s2 = sc;
    s2.prog = prog;
    s2.prog_mode = prog ? mode : 0;
    return s2;
  };
  if (n == 0) {
    c->launches++;
    return cuda_status(launch_header_only(out, codec, dtype, F, param_of(codec, f), out_size, st), "header");
  }
  switch (codec) {
    case CSWAP_CODEC_NONE:
      c->launches++;
      TRY(cuda_status(launch_none_compress(in, n, w, F, dtype, out, out_size, st), "none_compress"));
      return publish(st);
    case CSWAP_CODEC_ZVC: {
      uint64_t tiles = 0, aux = 0;
      zvc_compress_scratch(n, w, F, &tiles, &aux);
      Lease L(*c, st, tiles, aux);
      TRY(L.status);
      c->launches += 1;  // persistent compress (its accumulators clean up after themselves)
      const uint32_t ep = L.epoch();
      // per-frame publication from inside the persistent kernel only when asked (the D2H link
      // is idle, so the first frames' copies can overlap the rest of the compression); it costs
      // the kernel ~14 us (a gpu-scope acq_rel atomic per tile in the producer warp), so a
      // swap-out queued behind other copies has the kernel's last CTA publish every frame at
      // the end instead (no extra launch)
      static const bool end_kernel = getenv("CSWAP_ZVC_ENDPUB") && getenv("CSWAP_ZVC_ENDPUB")[0] == '0';  // A/B
      const uint32_t mode = frame_publish ? 1 : (end_kernel ? 0 : 2);
      Scratch sc = mode ? with_prog(L.b->sc, mode) : L.b->sc;
      // a timed group: the kernel also clocks itself into the timer's device slot (words 3, 4)
      sc.kclock = nullptr;
      if (t_pending && t_pending->stamps) {
        sc.kclock = t_pending->stamps + 3;
        t_pending->self_clocked = true;
      }
      return run_group(c, st, group_key(kGrpCompress, codec, dtype) | (mode == 0 && prog ? 1u << 21 : 0u),
                       [&](cudaStream_t gs) {
                         TRY(cuda_status(launch_zvc_compress(in, n, w, F, out, out_size, sc, ep, dtype, gs),
                                         "zvc_compress"));
                         return mode == 0 ? publish(gs) : CSWAP_OK;
                       });
    }
    case CSWAP_CODEC_RLE: {
      Lease L(*c, st, rle_tiles(n, w, F) + 2, uint64_t(K) + 2);
      TRY(L.status);
      c->launches += 4;
      const uint32_t ep = L.epoch();
      return run_group(c, st, group_key(kGrpCompress, codec, dtype), [&](cudaStream_t gs) {
        TRY(cuda_status(launch_rle_compress(in, n, w, F, out, out_size, L.b->sc, ep, dtype, gs), "rle_compress"));
        return publish(gs);
      });
    }
    case CSWAP_CODEC_CSR: {
      Lease L(*c, st, rle_tiles(n, w, F) + 2, uint64_t(K) + 2);
      TRY(L.status);
      c->launches += 4;
      const uint32_t ep = L.epoch();
      return run_group(c, st, group_key(kGrpCompress, codec, dtype), [&](cudaStream_t gs) {
        TRY(cuda_status(launch_csr_compress(in, n, w, F, f.csr_row, out, out_size, L.b->sc, ep, dtype, gs),
                        "csr_compress"));
        return publish(gs);
      });
    }
    case CSWAP_CODEC_LZ4: {
      const uint64_t blocks = lz4_scratch_bytes(n, w, F, f.lz4_block);
      uint8_t* slots = nullptr;
      CU(cudaMallocFromPoolAsync(reinterpret_cast<void**>(&slots), blocks, c->pool, st));
      const uint64_t bidx = uint64_t(K) * ((F * w + f.lz4_block - 1) / f.lz4_block);  // block index k*bpf + b
      cswap_status s;
      {
        Lease L(*c, st, bidx + 2, uint64_t(K) + 2);
        TRY(L.status);
        c->launches += 3;
        s = run_group(c, st, group_key(kGrpCompress, codec, dtype), [&](cudaStream_t gs) {
          TRY(cuda_status(launch_lz4_compress(in, n, w, F, f.lz4_block, out, out_size, slots, L.b->sc, dtype, gs),
                          "lz4_compress"));
          return publish(gs);
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
  uint8_t* host = nullptr;  // container (pinned pool): allocated at the codec's worst case, trimmed
  uint8_t* host_base = nullptr;  // the pool allocation `host` lies in (host = host_base + alignment pad)
  uint64_t bytes = 0;       // container bytes (valid once out_state != 0)
  uint64_t cap = 0;         // bytes allocated at `host`
  uint64_t n = 0;
  int dtype = 0, codec = 0;
  cswap_format fmt{};
  cswap_decision dec{};
  cudaEvent_t ev_out = nullptr, ev_in = nullptr;
  bool in_issued = false;
  uint8_t* slots = nullptr;  // pinned small slots: [64..68) swap-in error word
  uint32_t* err_slot() { return reinterpret_cast<uint32_t*>(slots + 64); }
  // swap-out state: 0 = the executor is still issuing the D2H copies, 1 = every copy is issued
  // and ev_out is recorded on the D2H stream, 2 = failed (out_err / out_msg)
  std::atomic<int> out_state{0};
  cswap_status out_err = CSWAP_OK;
  std::string out_msg;
  std::mutex m;
  std::condition_variable cv;
  // end offset of every frame in the container, as published by the compress kernels (the
  // executor's copy ranges; swap-in splits its H2D by these trusted values, never by the
  // host-resident frame table)
  std::vector<uint64_t> ends;
  // device target (NEXT-4b): the container lives in device memory of `target` (no host copy);
  // its size is written by the codec kernels into size_slot (pinned) and valid after ev_out
  int target = -1;
  uint8_t* dev = nullptr;
  uint64_t* size_slot() { return reinterpret_cast<uint64_t*>(slots); }
};

namespace {

struct OutJob {
  cswap_handle* h;
  uint8_t* staging;  // device container written by the compress group
  uint64_t* prog;    // host-mapped progress words (Scratch::prog)
  uint32_t K;
  cudaEvent_t done;  // recorded on the caller's stream after the compress group
  bool exact_host;   // frames arrive all at once: allocate the host container at its exact size
  uint64_t cap;      // staging bytes (the codec's worst case)
  uint8_t* staging_base;  // the pool allocation (staging = staging_base + alignment pad)
};

// DMA alignment: a D2H copy whose host destination is not 64-byte aligned runs at 52.3 GB/s,
// an aligned one at 57.1 (tools/d2h_step_probe.py: the same 784 MiB copy into the library's pinned
// container at its 80-byte data offset vs into a torch pinned tensor).  Containers are therefore
// placed in their pinned allocation so that `h->host` has a chosen residue mod 256 (the staging
// buffer's, or the raw tensor's minus the data offset), and copies start at 256-aligned addresses.
constexpr uintptr_t kDmaAlign = 256;
// a swap-out whose frames are published at the end of its group: the group writes the progress
// words to device memory and the progress stream copies them to the host (CSWAP_DEV_PROG=0: the
// group stores them to host-mapped memory itself, A/B)
#ifndef CSWAP_DEV_PROG
#define CSWAP_DEV_PROG 1
#endif
constexpr bool kDevProg = CSWAP_DEV_PROG != 0;
bool alloc_host(Ctx* c, cswap_handle* h, uint64_t bytes, uintptr_t residue) {
  h->host_base = c->pinned.alloc(bytes + kDmaAlign);
  if (!h->host_base) {
    h->host = nullptr;
    return false;
  }
  h->host = h->host_base + ((residue - reinterpret_cast<uintptr_t>(h->host_base)) & (kDmaAlign - 1));
  return true;
}
inline uintptr_t addr(const void* p) { return reinterpret_cast<uintptr_t>(p); }

void finish_out(cswap_handle* h, int state, cswap_status err, const std::string& msg) {
  {
    std::lock_guard<std::mutex> lk(h->m);
    h->out_err = err;
    h->out_msg = msg;
    h->out_state.store(state);
  }
  h->cv.notify_all();
}

// Block until the executor has issued every D2H copy of h (or failed).
cswap_status wait_out(cswap_handle* h) {
  if (h->out_state.load() == 0) {
    std::unique_lock<std::mutex> lk(h->m);
    h->cv.wait(lk, [&] { return h->out_state.load() != 0; });
  }
  if (h->out_state.load() == 2) return fail(h->out_err, "swap-out failed: %s", h->out_msg.c_str());
  return CSWAP_OK;
}

// Header + frame table of h's container, written on the host from the frame
// ends: byte-identical to what the codec kernels write into the device container (the tests
// compare the whole host container with the oracle), and it saves one small D2H per swap.
void write_host_header(cswap_handle* h) {
  const uint64_t F = h->fmt.frame_elems, n = h->n;
  const uint32_t K = uint32_t((n + F - 1) / F);
  const uint64_t ds = al16(64 + 8ull * K), total = K ? h->ends.back() : ds;
  std::memset(h->host, 0, ds);
  std::memcpy(h->host, "CSWP", 4);
  const uint16_t ver = 1;
  std::memcpy(h->host + 4, &ver, 2);
  h->host[6] = uint8_t(h->codec);
  h->host[7] = uint8_t(h->dtype);
  const uint32_t param = param_of(h->codec, h->fmt);
  std::memcpy(h->host + 8, &n, 8);
  std::memcpy(h->host + 16, &F, 8);
  std::memcpy(h->host + 24, &K, 4);
  std::memcpy(h->host + 28, &param, 4);
  std::memcpy(h->host + 32, &total, 8);
  uint64_t prev = ds;
  for (uint32_t k = 0; k < K; k++) {
    const uint64_t fb = h->ends[k] - prev;
    std::memcpy(h->host + 64 + 8ull * k, &fb, 8);
    prev = h->ends[k];
  }
}

// The executor's work for one swap-out: poll the progress words the compress group publishes
// into host-mapped memory and hand each newly completed run of frames to the copy engine
// (frame k's D2H overlaps the compression of frames k+1..), then the header + frame table, then
// record ev_out.  No event is recorded between the frame copies (each record would stall the
// D2H stream ~30 us behind the link's write queue, tools/event_probe.cu).
// pipeline granularities (bytes): environment override (read per call, for the A/B probes) or
// the default of 32 MiB
uint64_t env_bytes(const char* name, uint64_t dflt) {
  const char* e = getenv(name);
  return e ? uint64_t(atof(e) * double(1 << 20)) : dflt;
}

void run_out_job(Ctx* c, OutJob* j) {
  cswap_handle* h = j->h;
  const uint64_t min_copy = env_bytes("CSWAP_COPY_MB", uint64_t(32) << 20);  // D2H copy granularity
  const uint64_t ds = al16(64 + 8ull * j->K);
  uint64_t pos = ds;
  uint32_t k = 0;
  int idle = 0;
  bool group_done = false;
  cswap_status err = CSWAP_OK;
  std::string msg;
  h->ends.clear();
  h->ends.reserve(j->K);
  const volatile uint64_t* prog = j->prog;
  uint32_t k_ready = 0;  // frames whose end offset is known (h->ends[0 .. k_ready))
  while (k < j->K) {
    while (k_ready < j->K) {
      const uint64_t v = prog[k_ready];
      if (!(v & kProgReady)) break;
      const uint64_t e = v & ~kProgReady;
      if (e < (k_ready ? h->ends.back() : ds) || e > j->cap || (e & 15)) {
        err = CSWAP_ERR_CUDA;
        char b[256];
        snprintf(b, sizeof(b),
                 "inconsistent progress word from the compress kernel (codec %d, frame %u of %u: end %llu, "
                 "previous %llu, capacity %llu)",
                 h->codec, k_ready, j->K, (unsigned long long)e,
                 (unsigned long long)(k_ready ? h->ends.back() : ds), (unsigned long long)j->cap);
        msg = b;
        break;
      }
      h->ends.push_back(e);
      k_ready++;
    }
    if (err != CSWAP_OK) break;
    if (j->exact_host && k_ready == j->K && !h->host) {
      // every frame is published at once (publication after the codec's last kernel): pin the
      // container at its exact size (no worst-case allocation: RLE / CSR reserve 2-3x raw)
      alloc_host(c, h, h->ends.back(), addr(j->staging));  // host == staging (mod 256)
      h->cap = h->ends.back();
      if (!h->host) {
        err = CSWAP_ERR_NOMEM;
        msg = "pinned alloc of the container failed";
        break;
      }
    }
    if (k_ready > k && (!j->exact_host || k_ready == j->K)) {  // exact_host: the whole container at once
      const uint64_t end = h->ends[k_ready - 1];
      // copy granularity: every D2H copy costs a few us of DMA ramp and tail, so published frames
      // are coalesced until `min_copy` bytes are ready -- unless the D2H stream is idle (then any
      // frame goes at once: this is what overlaps a tensor's first frames with its compression)
      // or every frame is published
      if (k_ready < j->K && end - pos < min_copy && cudaStreamQuery(c->s_d2h) == cudaErrorNotReady) {
        std::this_thread::yield();
        continue;
      }
      // start at the 256-aligned address at or below pos (re-copying up to 255 bytes the previous
      // copy already moved: the staging bytes are final), never below the data start
      const uint64_t start = pos - std::min<uint64_t>(pos - ds, addr(j->staging + pos) & (kDmaAlign - 1));
      if (end > pos &&
          cudaMemcpyAsync(h->host + start, j->staging + start, end - start, cudaMemcpyDeviceToHost, c->s_d2h) !=
              cudaSuccess) {
        err = CSWAP_ERR_CUDA;
        msg = cudaGetErrorString(cudaGetLastError());
        break;
      }
      pos = end;
      k = k_ready;
      idle = 0;
      continue;
    }
    if (group_done) {  // the group finished (its writes to mapped memory are visible) but not all frames
      err = CSWAP_ERR_CUDA;
      msg = "compress finished without publishing every frame";
      break;
    }
    const cudaError_t e = cudaEventQuery(j->done);
    if (e == cudaSuccess) {
      group_done = true;  // one more pass over the progress words
      continue;
    }
    if (e != cudaErrorNotReady) {
      err = CSWAP_ERR_CUDA;
      msg = cudaGetErrorString(e);
      break;
    }
    // nothing new yet: spin briefly (a frame completes every few us while the kernel runs),
    // then back off so that a long queue of pending compresses does not burn a core
    if (++idle < 4096) std::this_thread::yield();
    else std::this_thread::sleep_for(std::chrono::microseconds(20));
  }
  if (err == CSWAP_OK && !h->host) {  // n = 0: a header-only container
    alloc_host(c, h, pos, 0);
    h->cap = pos;
    if (!h->host) {
      err = CSWAP_ERR_NOMEM;
      msg = "pinned alloc of the container failed";
    }
  }
  if (err == CSWAP_OK) write_host_header(h);
  // staging is freed on the D2H stream behind the copies; when nothing waited for the kernels
  // (a failure, or n = 0 with no frame to publish) the free is ordered behind the group itself
  if (err != CSWAP_OK || j->K == 0) cudaStreamWaitEvent(c->s_d2h, j->done, 0);
  if (err != CSWAP_OK) cudaEventSynchronize(j->done);  // the kernels may still write progress words
  cudaFreeAsync(j->staging_base, c->s_d2h);
  cudaEventRecord(h->ev_out, c->s_d2h);
  cudaEventDestroy(j->done);
  c->small.free(reinterpret_cast<uint8_t*>(j->prog));  // the kernel has written its last word
  if (err == CSWAP_OK) {
    h->bytes = pos;
    c->pinned.shrink(h->host_base, uint64_t(h->host - h->host_base) + pos);
    h->cap = pos;
  }
  finish_out(h, err == CSWAP_OK ? 1 : 2, err, msg);
}

void executor_main(Ctx* c) {
  cudaSetDevice(c->device);
  for (;;) {
    OutJob* j = nullptr;
    {
      std::unique_lock<std::mutex> lk(c->qm);
      c->qcv.wait(lk, [&] { return c->stop || !c->q.empty(); });
      if (c->q.empty()) return;  // stop requested and drained
      j = c->q.front();
    }
    run_out_job(c, j);
    {
      std::lock_guard<std::mutex> lk(c->qm);
      c->q.pop_front();
    }
    delete j;
  }
}

void enqueue_out(Ctx* c, OutJob* j) {
  {
    std::lock_guard<std::mutex> lk(c->qm);
    c->q.push_back(j);
  }
  c->qcv.notify_one();
}

}  // namespace

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
  CU(cudaStreamCreateWithFlags(&c->s_h2d2, cudaStreamNonBlocking));
  CU(cudaStreamCreateWithFlags(&c->s_prog, cudaStreamNonBlocking));
  for (auto& b : c->blocks) {
    CU(cudaEventCreateWithFlags(&b.ev, cudaEventDisableTiming));
    TRY(ensure_block(b, 1 << 16, 1 << 12));
  }
  // a private pool ("memory pool"): staging memory stays reserved between swaps up
  // to a bounded threshold (CSWAP_POOL_KEEP_MB, default 16 GiB of the 180: a training step's
  // worst-case staging in flight; trimming below it made every step re-map pool memory, which
  // stalled the forward pass) and the process's default pool is left as the
  // application configured it
  cudaMemPoolProps pp = {};
  pp.allocType = cudaMemAllocationTypePinned;
  pp.location.type = cudaMemLocationTypeDevice;
  pp.location.id = device;
  CU(cudaMemPoolCreate(&c->pool, &pp));
  uint64_t keep = uint64_t(16384) << 20;
  if (const char* e = getenv("CSWAP_POOL_KEEP_MB")) keep = uint64_t(atoll(e)) << 20;
  CU(cudaMemPoolSetAttribute(c->pool, cudaMemPoolAttrReleaseThreshold, &keep));
  CU(cudaMalloc(&c->dev_err, 64));
  CU(cudaMemset(c->dev_err, 0, 64));
  CU(cudaMalloc(&c->dev_sink, 64));
  CU(cudaMalloc(&c->dev_stamps, 8ull * Ctx::kStampWords * Ctx::kStampSlots));
  if (const char* e = getenv("CSWAP_PINNED_CHUNK_MB")) c->pinned.chunk_bytes = uint64_t(atoll(e)) << 20;
  c->small.chunk_bytes = uint64_t(1) << 20;
  c->calib = builtin_calib();
  c->fmt = cswap_format{uint64_t(1) << 22, 1024, 65536};
  c->exec = std::thread(executor_main, c);
  g_ctx = c;
  return CSWAP_OK;
}

cswap_status cswap_shutdown(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g_ctx) return CSWAP_OK;
  Ctx* c = g_ctx;
  {
    std::lock_guard<std::mutex> lk(c->qm);
    c->stop = true;
  }
  c->qcv.notify_all();
  if (c->exec.joinable()) c->exec.join();  // drains the queued swap-outs first
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
    cudaFree(b.sc.zacc);
    cudaEventDestroy(b.ev);
  }
  cudaFree(c->dev_err);
  cudaFree(c->dev_sink);
  cudaFree(c->dev_stamps);
  cudaMemPoolDestroy(c->pool);
  if (c->tpool) cudaMemPoolDestroy(c->tpool);
  cudaStreamDestroy(c->s_d2h);
  cudaStreamDestroy(c->s_h2d);
  cudaStreamDestroy(c->s_h2d2);
  cudaStreamDestroy(c->s_prog);
  c->pinned.destroy();
  c->small.destroy();
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
  if (!zvc_set_launch(grid, variant)) return fail(CSWAP_ERR_INVALID, "variant %d outside -1..9", int(variant));
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

}  // extern "C"

namespace {
// decompress a whole container (device memory) into d_out on st; device-side validation
// failures are merged into *user_err (device-visible word)
cswap_status decompress_impl(Ctx* c, const uint8_t* inb, uint64_t in_size, void* d_out, uint64_t n, int dtype,
                             int codec, const cswap_format& f, uint32_t* user_err, cudaStream_t st) {
  const int w = width(dtype);
  const uint64_t F = f.frame_elems;
  const uint32_t K = uint32_t((n + F - 1) / F);
  Lease L(*c, st, decompress_tiles(n, w, f), decompress_aux(n, w, f));
  TRY(L.status);
  // kernels flag errors in the lease's device word (never in host-mapped memory: every CTA
  // reads it); the word is merged into the caller's at the end
  uint32_t* e = L.b->sc.err;
  uint8_t* tmp = nullptr;
  const uint64_t tmp_bytes = n ? decompress_tmp_bytes(codec, n, f, 0, K) : 0;
  if (tmp_bytes) CU(cudaMallocFromPoolAsync(reinterpret_cast<void**>(&tmp), tmp_bytes, c->pool, st));
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
}  // namespace

extern "C" {

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
  return decompress_impl(c, static_cast<const uint8_t*>(in), in_size, d_out, n, dtype, codec, f,
                         err ? err : c->dev_err, static_cast<cudaStream_t>(stream));
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
  uint8_t* slot = c->small.alloc(256);
  if (!slot) return fail(CSWAP_ERR_NOMEM, "pinned alloc failed");
  volatile uint64_t* counts = reinterpret_cast<volatile uint64_t*>(slot);
  counts[0] = counts[1] = counts[2] = 0;
  static std::atomic<uint32_t> tags{0};
  uint32_t tag = 0;
  while (tag == 0) tag = tags.fetch_add(1) & 0xFFFFu;  // nonzero, differs from the slot's last use
  cswap_status s = CSWAP_OK;
  {
    Lease L(*c, st, 1024, 1024);
    s = L.status;
    if (s == CSWAP_OK) {
      Timer tm(c, st);
      c->launches++;
      s = cuda_status(launch_probe(d_in, n, w, reinterpret_cast<uint64_t*>(slot), tag, L.b->sc, L.epoch(), st),
                      "probe");
      tm.commit(0, 2, std::min<uint64_t>(n, 262144) * w, 0);
    }
  }
  // wait for the three tagged counts in mapped memory.  No completion event: an event record
  // costs the stream ~25-35 us while a copy engine streams over PCIe (tools/event_probe.cu), the
  // probe kernel itself ~7 us.  A failed or missing kernel is caught through the stream state.
  auto ready = [&] { return (counts[0] & 0xFFFF) == tag && (counts[1] & 0xFFFF) == tag && (counts[2] & 0xFFFF) == tag; };
  for (uint64_t spin = 0; s == CSWAP_OK && !ready(); spin++) {
    if ((spin & 1023) == 1023) {
      const cudaError_t e = cudaStreamQuery(st);
      if (e == cudaSuccess && !ready()) s = fail(CSWAP_ERR_CUDA, "probe finished without publishing its counts");
      else if (e != cudaSuccess && e != cudaErrorNotReady) s = cuda_status(e, "probe");
    }
    if (spin > 4096) std::this_thread::yield();
  }
  if (s == CSWAP_OK) {
    const bool single = n <= 262144;
    out->zeros = counts[0] >> 16;
    out->zero_runs = counts[1] >> 16;
    out->boundaries = counts[2] >> 16;
    out->samples = single ? n : 262144;
    out->pairs = out->samples - (single ? 1 : 1024);
  }
  if (s == CSWAP_OK) c->small.free(slot);  // (on failure the slot is leaked: the kernel may still write it)
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

// ---- swap target (NEXT-4b) ------------------------------------------------------------------
cswap_status cswap_set_swap_target(int device) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  std::lock_guard<std::mutex> lk(c->cfg_m);
  if (device < 0) {
    c->target = -1;
    return CSWAP_OK;
  }
  int count = 0;
  CU(cudaGetDeviceCount(&count));
  if (device >= count) return fail(CSWAP_ERR_INVALID, "device %d does not exist (%d visible)", device, count);
  if (device != c->device) {
    int ok = 0;
    CU(cudaDeviceCanAccessPeer(&ok, c->device, device));
    if (!ok) return fail(CSWAP_ERR_UNSUPPORTED, "device %d cannot reach device %d by peer access", c->device, device);
    const cudaError_t e = cudaDeviceEnablePeerAccess(device, 0);
    if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cuda_status(e, "enable peer access");
    cudaGetLastError();
  }
  if (c->tpool) {
    cudaMemPoolDestroy(c->tpool);
    c->tpool = nullptr;
  }
  // containers live in a pool located on the target device and accessible from this one: the
  // codec kernels store into it (over NVLink for a peer) and the decoders read from it
  cudaMemPoolProps pp = {};
  pp.allocType = cudaMemAllocationTypePinned;
  pp.location.type = cudaMemLocationTypeDevice;
  pp.location.id = device;
  CU(cudaMemPoolCreate(&c->tpool, &pp));
  if (device != c->device) {
    cudaMemAccessDesc ad = {};
    ad.location.type = cudaMemLocationTypeDevice;
    ad.location.id = c->device;
    ad.flags = cudaMemAccessFlagsProtReadWrite;
    CU(cudaMemPoolSetAccess(c->tpool, &ad, 1));
  }
  uint64_t keep = uint64_t(4096) << 20;
  CU(cudaMemPoolSetAttribute(c->tpool, cudaMemPoolAttrReleaseThreshold, &keep));
  c->target = device;
  return CSWAP_OK;
}

cswap_status cswap_get_swap_target(int* device) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  if (!device) return fail(CSWAP_ERR_INVALID, "device is NULL");
  std::lock_guard<std::mutex> lk(c->cfg_m);
  *device = c->target;
  return CSWAP_OK;
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
  h->slots = c->small.alloc(256);
  if (!h->slots) {
    delete h;
    return fail(CSWAP_ERR_NOMEM, "pinned alloc failed");
  }
  auto bail = [&](cswap_status s) {
    finish_out(h, 2, s, "swap-out not issued");
    cswap_handle_free(h);
    return s;
  };
  if (cudaEventCreateWithFlags(&h->ev_out, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&h->ev_in, cudaEventDisableTiming) != cudaSuccess)
    return bail(fail(CSWAP_ERR_CUDA, "event create failed"));
  int use = codec;
  if (codec == CSWAP_CODEC_AUTO) {
    // the selector runs on the host, so AUTO waits for the probe's counts:
    // the one host synchronisation of the swap-out path.  Fixed codecs (or a replayed plan,
    // NEXT-2) never block the caller.
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
  const uint64_t ds = al16(64 + 8ull * K);
  cudaMemPool_t tpool = nullptr;
  {
    std::lock_guard<std::mutex> lk(c->cfg_m);
    h->target = c->target;
    tpool = c->tpool;
  }
  if (h->target >= 0) {
    // device target (NEXT-4b): the codec kernels write the container straight into the target's
    // memory -- peer-mapped stores over NVLink for a peer -- sized for the codec's worst case;
    // everything is ordered on the caller's stream, nothing waits on the host
    const uint64_t cap = max_size(n, w, use, f);
    if (cudaMallocFromPoolAsync(reinterpret_cast<void**>(&h->dev), cap, tpool, st) != cudaSuccess)
      return bail(fail(CSWAP_ERR_NOMEM, "container of %llu B on device %d failed", (unsigned long long)cap, h->target));
    h->cap = cap;
    cswap_status s;
    {
      Timer tm(c, st);
      s = do_compress(c, d_in, n, dtype, use, f, h->dev, h->size_slot(), st);
      if (s == CSWAP_OK) tm.commit(use, 0, n * uint64_t(w), 0);
    }
    if (s == CSWAP_OK && cudaEventRecord(h->ev_out, st) != cudaSuccess) s = fail(CSWAP_ERR_CUDA, "event record");
    if (s != CSWAP_OK) {
      cudaFreeAsync(h->dev, st);
      h->dev = nullptr;
      return bail(s);
    }
    finish_out(h, 1, CSWAP_OK, "");
    *out = h;
    return CSWAP_OK;
  }
  if (use == CSWAP_CODEC_NONE) {
    // raw offload (vDNN): the host writes header + frame table, the copy engine
    // moves the tensor's bytes straight into the frames after the caller's stream reaches here
    const uint64_t cap = max_size(n, w, CSWAP_CODEC_NONE, f);
    alloc_host(c, h, cap, addr(d_in) - ds);  // host + ds == d_in (mod 256): aligned raw copies
    if (!h->host) return bail(fail(CSWAP_ERR_NOMEM, "pinned alloc of %llu B failed", (unsigned long long)cap));
    h->cap = cap;
    const uint64_t tail = ds + uint64_t(w) * n;
    std::memset(h->host + tail, 0, cap - tail);  // frame padding
    uint64_t total = ds;
    for (uint32_t k = 0; k < K; k++) {
      total += al16(uint64_t(w) * std::min<uint64_t>(F, n - uint64_t(k) * F));
      h->ends.push_back(total);
    }
    write_host_header(h);
    h->bytes = total;
    if (n) {
      cudaEvent_t ready;
      if (cudaEventCreateWithFlags(&ready, cudaEventDisableTiming) != cudaSuccess)
        return bail(fail(CSWAP_ERR_CUDA, "event create failed"));
      const bool ok = cudaEventRecord(ready, st) == cudaSuccess && cudaStreamWaitEvent(c->s_d2h, ready, 0) == cudaSuccess &&
                      cudaMemcpyAsync(h->host + ds, d_in, uint64_t(w) * n, cudaMemcpyDeviceToHost, c->s_d2h) == cudaSuccess;
      cudaEventDestroy(ready);
      if (!ok) return bail(fail(CSWAP_ERR_CUDA, "raw offload failed"));
    }
    cudaEventRecord(h->ev_out, c->s_d2h);
    finish_out(h, 1, CSWAP_OK, "");
    *out = h;
    return CSWAP_OK;
  }
  // compressed offload ("compression in parallel before swapping"; Fig. 2): the
  // codec writes the container into device staging sized for its worst case and publishes each
  // finished frame; the executor thread copies frames to the pinned host container as they are
  // published.  Nothing here waits for the device.
  const uint64_t cap = max_size(n, w, use, f);
  // staging placed so that its data start (staging + ds) is 256-aligned: the first copy of every
  // container starts aligned, later copies start at aligned addresses at or below their frame
  uint8_t* staging_base = nullptr;
  const uint64_t prog_bytes = 8ull * std::max<uint32_t>(K, 1);
  if (cudaMallocFromPoolAsync(reinterpret_cast<void**>(&staging_base), cap + 2 * kDmaAlign + prog_bytes, c->pool,
                              st) != cudaSuccess)
    return bail(fail(CSWAP_ERR_NOMEM, "device staging of %llu B failed", (unsigned long long)cap));
  uint8_t* staging = staging_base + ((uintptr_t(0) - ds - addr(staging_base)) & (kDmaAlign - 1));
  // device copy of the progress words, after the container (published by the group, copied to
  // the host words on the progress stream once the group is done)
  uint64_t* dprog = reinterpret_cast<uint64_t*>(staging + ((cap + kDmaAlign - 1) & ~uint64_t(kDmaAlign - 1)));
  // per-frame publication pays only when the D2H link would otherwise wait for this tensor's
  // compression (nothing queued ahead of it); CSWAP_FRAME_PUBLISH=0/1 forces it off/on.  Only
  // ZVC publishes from inside its kernel; then the host container is pinned at the worst case
  // (1.03x raw) up front, else the executor pins it at its exact size once it is known.
  bool frame_publish;
  if (const char* e = getenv("CSWAP_FRAME_PUBLISH")) {
    frame_publish = e[0] == '1';
  } else {
    std::lock_guard<std::mutex> lk(c->qm);
    frame_publish = c->q.empty() && cudaStreamQuery(c->s_d2h) == cudaSuccess;
  }
  frame_publish = frame_publish && use == CSWAP_CODEC_ZVC;
  if (frame_publish) {
    alloc_host(c, h, cap, addr(staging));  // host == staging (mod 256)
    h->cap = cap;
  }
  uint64_t* prog = reinterpret_cast<uint64_t*>(c->small.alloc(8ull * std::max<uint32_t>(K, 1)));
  if ((frame_publish && !h->host) || !prog) {
    cudaFreeAsync(staging_base, st);
    c->small.free(reinterpret_cast<uint8_t*>(prog));
    return bail(fail(CSWAP_ERR_NOMEM, "pinned alloc of %llu B failed", (unsigned long long)cap));
  }
  std::memset(prog, 0, 8ull * std::max<uint32_t>(K, 1));
  cswap_status s;
  cudaEvent_t done = nullptr;
  {
    Timer tm(c, st);
    // the container size goes to the timer's pinned slot when timing (read at collection), else
    // to a device word nobody reads (the executor takes the size from the progress words)
    uint64_t* osz = tm.stamps ? tm.stamps + 2 : c->dev_sink;
    // frames published one by one from inside the kernel go straight to the host words; a group
    // that publishes at its end writes device words, copied below
    s = do_compress(c, d_in, n, dtype, use, f, staging, osz, st, (frame_publish || !kDevProg) ? prog : dprog,
                    frame_publish);
    if (s == CSWAP_OK) tm.commit(use, 0, n * uint64_t(w), 0);
  }
  if (s == CSWAP_OK && (cudaEventCreateWithFlags(&done, cudaEventDisableTiming) != cudaSuccess ||
                        cudaEventRecord(done, st) != cudaSuccess))
    s = fail(CSWAP_ERR_CUDA, "event record failed");
  if (s == CSWAP_OK && !frame_publish && kDevProg) {
    // the progress words reach the host after the group: `done` is re-recorded behind the copy,
    // so "group done" still implies "every word visible" for the executor
    if (cudaStreamWaitEvent(c->s_prog, done, 0) != cudaSuccess ||
        cudaMemcpyAsync(prog, dprog, prog_bytes, cudaMemcpyDeviceToHost, c->s_prog) != cudaSuccess ||
        cudaEventRecord(done, c->s_prog) != cudaSuccess)
      s = fail(CSWAP_ERR_CUDA, "progress copy failed");
  }
  if (s != CSWAP_OK) {
    if (done) cudaEventDestroy(done);
    cudaFreeAsync(staging_base, st);
    cudaStreamSynchronize(st);  // the group may have been partly enqueued: prog is still referenced
    c->small.free(reinterpret_cast<uint8_t*>(prog));
    return bail(s);
  }
  enqueue_out(c, new OutJob{h, staging, prog, K, done, !frame_publish, cap, staging_base});
  *out = h;
  return CSWAP_OK;
}

cswap_status cswap_swap_in(cswap_handle* h, void* d_out, void* stream) {
  if (!h) return fail(CSWAP_ERR_INVALID, "handle is NULL");
  Ctx* c = h->ctx;
  const int w = width(h->dtype);
  if (h->n) TRY(check_common(d_out, "d_out"));
  TRY(wait_out(h));  // the executor has issued the D2H copies: frame ranges known, ev_out recorded
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const cswap_format& f = h->fmt;
  const uint64_t F = f.frame_elems, n = h->n;
  const uint32_t K = uint32_t((n + F - 1) / F);
  const uint64_t ds = al16(64 + 8ull * K);
  h->in_issued = true;
  *h->err_slot() = 0;
  if (h->dev) {  // device target: decode straight from the container (peer loads over NVLink)
    CU(cudaStreamWaitEvent(st, h->ev_out, 0));  // same stream unless the caller switched streams
    TRY(decompress_impl(c, h->dev, h->cap, d_out, n, h->dtype, h->codec, f, h->err_slot(), st));
    CU(cudaEventRecord(h->ev_in, st));
    return CSWAP_OK;
  }
  if (n == 0) return cudaEventRecord(h->ev_in, st) == cudaSuccess ? CSWAP_OK : fail(CSWAP_ERR_CUDA, "record");
  if (h->ends.size() != K || h->ends.back() != h->bytes)
    return fail(CSWAP_ERR_CORRUPT, "frame ranges of the handle are inconsistent");
  // the H2D copies are ordered after the D2H on the device (no host wait for the swap-out)
  CU(cudaStreamWaitEvent(c->s_h2d, h->ev_out, 0));
  if (h->codec == CSWAP_CODEC_NONE) {
    cudaEvent_t ready;
    CU(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming));
    cswap_status s = CSWAP_OK;
    if (cudaEventRecord(ready, st) != cudaSuccess || cudaStreamWaitEvent(c->s_h2d, ready, 0) != cudaSuccess ||
        cudaMemcpyAsync(d_out, h->host + ds, uint64_t(w) * n, cudaMemcpyHostToDevice, c->s_h2d) != cudaSuccess ||
        cudaEventRecord(h->ev_in, c->s_h2d) != cudaSuccess || cudaStreamWaitEvent(st, h->ev_in, 0) != cudaSuccess)
      s = fail(CSWAP_ERR_CUDA, "raw prefetch failed");
    cudaEventDestroy(ready);
    return s;
  }
  CU(cudaStreamWaitEvent(c->s_h2d2, h->ev_out, 0));
  // pipelined prefetch in groups of whole frames (R7, R22; the cost model's G): group g's H2D
  // overlaps the decompression of group g-1.  Staging is allocated on the first copy stream,
  // which the second copy stream follows; consecutive groups alternate between the two streams.
  // staging == host (mod 256), and every H2D step starts at a 256-aligned address at or below
  // its first byte (re-reading up to 255 bytes of the previous step: identical values)
  uint8_t* staging_base = nullptr;
  if (cudaMallocFromPoolAsync(reinterpret_cast<void**>(&staging_base), h->bytes + kDmaAlign, c->pool, c->s_h2d) !=
      cudaSuccess)
    return fail(CSWAP_ERR_NOMEM, "swap-in staging of %llu B failed", (unsigned long long)h->bytes);
  uint8_t* staging = staging_base + ((addr(h->host) - addr(staging_base)) & (kDmaAlign - 1));
  std::vector<cudaEvent_t> evs;
  cswap_status s = CSWAP_OK;
  cudaEvent_t alloc_ev;
  CU(cudaEventCreateWithFlags(&alloc_ev, cudaEventDisableTiming));
  evs.push_back(alloc_ev);
  if (cudaEventRecord(alloc_ev, c->s_h2d) != cudaSuccess || cudaStreamWaitEvent(c->s_h2d2, alloc_ev, 0) != cudaSuccess)
    s = fail(CSWAP_ERR_CUDA, "stream order failed");
  // pipeline steps: runs of whole frames of >= min_group container bytes (one H2D copy + one
  // decode launch group each; a copy's DMA ramp / tail costs a few us, so the link runs at
  // 53.4 GB/s with one copy per 8 MiB frame and 54.7 with ~32 MiB copies)
  const uint64_t min_group = env_bytes("CSWAP_SWAPIN_GROUP_MB", uint64_t(32) << 20);
  const bool two_streams = !(getenv("CSWAP_SWAPIN_STREAMS") && getenv("CSWAP_SWAPIN_STREAMS")[0] == '1');
  std::vector<uint32_t> gk{0};
  {
    uint64_t start = 0;
    for (uint32_t k = 0; k < K; k++)
      if (h->ends[k] - start >= min_group || k + 1 == K) {
        gk.push_back(k + 1);
        start = h->ends[k];
      }
  }
  {
    Lease L(*c, st, decompress_tiles(n, w, f), decompress_aux(n, w, f));
    if (s == CSWAP_OK) s = L.status;
    uint32_t* e_dev = L.b->sc.err;  // device word; merged into the handle's pinned slot at the end
    uint64_t off = 0;
    uint32_t gi = 0;
    for (; gi + 1 < gk.size() && s == CSWAP_OK; gi++) {
      const uint32_t k0 = gk[gi], k1 = gk[gi + 1];
      const uint64_t end = h->ends[k1 - 1];  // trusted: published by the compress kernels
      if (end <= off || end > h->bytes) {
        s = fail(CSWAP_ERR_CORRUPT, "frame range out of bounds");
        break;
      }
      cudaStream_t cs = ((gi & 1) && two_streams) ? c->s_h2d2 : c->s_h2d;
      cudaEvent_t e;
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) {
        s = fail(CSWAP_ERR_CUDA, "event create");
        break;
      }
      evs.push_back(e);
      const uint64_t start = off - std::min<uint64_t>(off, addr(h->host + off) & (kDmaAlign - 1));
      if (cudaMemcpyAsync(staging + start, h->host + start, end - start, cudaMemcpyHostToDevice, cs) != cudaSuccess ||
          cudaEventRecord(e, cs) != cudaSuccess || cudaStreamWaitEvent(st, e, 0) != cudaSuccess) {
        s = fail(CSWAP_ERR_CUDA, "prefetch copy failed");
        break;
      }
      uint8_t* tmp = nullptr;
      const uint64_t tmp_bytes = decompress_tmp_bytes(h->codec, n, f, k0, k1);
      if (tmp_bytes && cudaMallocFromPoolAsync(reinterpret_cast<void**>(&tmp), tmp_bytes, c->pool, st) != cudaSuccess) {
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
  // every staging read is on st (the last decode); frees and the end event follow it there
  cudaFreeAsync(staging_base, st);
  cudaEventRecord(h->ev_in, st);
  for (auto e : evs) cudaEventDestroy(e);
  return s;
}

cswap_status cswap_handle_wait(cswap_handle* h) {
  if (!h) return fail(CSWAP_ERR_INVALID, "handle is NULL");
  TRY(wait_out(h));
  CU(cudaEventSynchronize(h->ev_out));
  if (h->in_issued) {
    CU(cudaEventSynchronize(h->ev_in));
    if (*h->err_slot()) return fail(CSWAP_ERR_CORRUPT, "swap-in validation failed");
  }
  return CSWAP_OK;
}

cswap_status cswap_handle_record_out(cswap_handle* h, void* stream) {
  if (!h) return fail(CSWAP_ERR_INVALID, "handle is NULL");
  TRY(wait_out(h));
  CU(cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), h->ev_out, 0));
  return CSWAP_OK;
}

cswap_status cswap_handle_query(const cswap_handle* hc, cswap_codec* codec, uint64_t* container_bytes,
                                const void** host_container, cswap_decision* decision) {
  if (!hc) return fail(CSWAP_ERR_INVALID, "handle is NULL");
  cswap_handle* h = const_cast<cswap_handle*>(hc);  // waiting on the handle's state is not a change
  if (codec) *codec = cswap_codec(h->codec);
  if (decision) *decision = h->dec;
  if (container_bytes || host_container) {
    TRY(wait_out(h));
    if (h->dev && !h->bytes) {  // device target: the size the codec kernels wrote
      CU(cudaEventSynchronize(h->ev_out));
      h->bytes = *reinterpret_cast<volatile uint64_t*>(h->size_slot());
    }
    if (container_bytes) *container_bytes = h->bytes;
    if (host_container) *host_container = h->host;
  }
  return CSWAP_OK;
}

void cswap_handle_free(cswap_handle* h) {
  if (!h) return;
  wait_out(h);  // the executor no longer touches h
  if (h->ev_out) cudaEventSynchronize(h->ev_out);
  if (h->ev_in && h->in_issued) cudaEventSynchronize(h->ev_in);
  if (h->ev_out) cudaEventDestroy(h->ev_out);
  if (h->ev_in) cudaEventDestroy(h->ev_in);
  if (h->dev) cudaFreeAsync(h->dev, h->ctx->s_d2h);  // every use is complete (events above)
  h->ctx->pinned.free(h->host_base);
  h->ctx->small.free(h->slots);
  delete h;
}

cswap_status cswap_handle_copy_container(cswap_handle* h, void* dst, uint64_t cap, void* stream) {
  if (!h || !dst) return fail(CSWAP_ERR_INVALID, "bad arguments");
  uint64_t bytes = 0;
  TRY(cswap_handle_query(h, nullptr, &bytes, nullptr, nullptr));
  if (cap < bytes) return fail(CSWAP_ERR_CAPACITY, "cap %llu < %llu", (unsigned long long)cap, (unsigned long long)bytes);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  CU(cudaStreamWaitEvent(st, h->ev_out, 0));
  CU(cudaMemcpyAsync(dst, h->dev ? static_cast<const void*>(h->dev) : h->host, bytes, cudaMemcpyDefault, st));
  CU(cudaStreamSynchronize(st));
  return CSWAP_OK;
}

cswap_status cswap_release_cached(uint64_t keep_bytes) {
  Ctx* c = nullptr;
  TRY(need_ctx(&c));
  CU(cudaDeviceSynchronize());
  CU(cudaMemPoolTrimTo(c->pool, keep_bytes));
  if (c->tpool) CU(cudaMemPoolTrimTo(c->tpool, keep_bytes));
  c->pinned.release_empty();
  c->small.release_empty();
  return CSWAP_OK;
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
    uint64_t t[Ctx::kStampWords] = {};  // written by the group's kernels, complete once e.b is
    if (e.stamps && cudaMemcpy(t, e.stamps, sizeof(t), cudaMemcpyDeviceToHost) == cudaSuccess) {
      if (e.stamped) e.r.device_ms = (t[0] && t[1] > t[0]) ? double(t[1] - t[0]) * 1e-6 : 0.0;
      if (e.self_clocked) e.r.kernel_ms = t[4] > t[3] ? double(t[4] - t[3]) * 1e-6 : 0.0;
      if (!e.r.comp_bytes) e.r.comp_bytes = t[2];  // swap-out compress: container size
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
