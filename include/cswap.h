/*
 * cswap.h — C ABI of the B200-native CSWAP hot path (libcswap.so).
 *
 * CSWAP (Chen et al., CLUSTER'21, /root/reference/PAPER.md) swaps sparse activation tensors
 * between GPU and host memory and compresses them on the GPU when that is cost-effective:
 *   - four lossless codecs: ZVC, RLE, CSR, LZ4 (§IV-E);
 *   - swap-out = compress + D2H to pinned host memory, swap-in = H2D + decompress
 *     (PAPER.md:120, :228, §IV-A/§V; Fig. 2, :64-:72);
 *   - a cost model that decides per tensor whether and how to compress
 *     (§IV-B, Eq. 1-4; codec choice :30; time model §IV-C :164-168).
 * The byte format of every container is "canonical container v1".
 *
 * Conventions (all functions):
 *   - Plain C types only.  `stream` is a cudaStream_t passed as void* (NULL = legacy default).
 *   - Device pointers must be CUDA device memory (or host-mapped pinned memory where noted) of
 *     the device given to cswap_init; tensor and container buffers must be 16-byte aligned.
 *   - Every call returns a cswap_status and never aborts.  Host-detectable misuse returns
 *     synchronously; asynchronous kernel-side problems (corrupt containers) are reported through
 *     a device-visible error word (cswap_decompress) or by cswap_handle_wait (swaps).
 *   - cswap_last_error() gives a thread-local human-readable detail for the last failure.
 *   - Elements are raw 32-bit (f32) or 16-bit (f16, bf16) words; "zero" means all bits zero
 *     (R1), so NaN payloads, -0.0 and denormals round-trip bit-exactly.
 */
#ifndef CSWAP_H
#define CSWAP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  CSWAP_OK = 0,
  CSWAP_ERR_INVALID = 1,     /* bad argument (null pointer, misalignment, bad dtype/codec/format) */
  CSWAP_ERR_CUDA = 2,        /* a CUDA runtime call failed; see cswap_last_error() */
  CSWAP_ERR_NOMEM = 3,       /* device or pinned host allocation failed */
  CSWAP_ERR_CAPACITY = 4,    /* output buffer smaller than cswap_max_compressed_size() */
  CSWAP_ERR_CORRUPT = 5,     /* container failed validation */
  CSWAP_ERR_UNSUPPORTED = 6, /* valid request this build does not implement */
  CSWAP_ERR_NOT_READY = 7    /* library not initialised */
} cswap_status;

typedef enum {
  CSWAP_CODEC_NONE = 0, /* raw copy (vDNN-style uncompressed swap) */
  CSWAP_CODEC_ZVC = 1,  /* zero-value compression: 1-bit-per-element bitmap + non-zeros */
  CSWAP_CODEC_RLE = 2,  /* run-length encoding: (length, value) per maximal run */
  CSWAP_CODEC_CSR = 3,  /* compressed sparse rows of C elements */
  CSWAP_CODEC_LZ4 = 4,  /* LZ4 block format, canonical greedy parse */
  CSWAP_CODEC_AUTO = 255 /* cswap_swap_out only: probe + cost model pick one */
} cswap_codec;

typedef enum { CSWAP_F32 = 0, CSWAP_F16 = 1, CSWAP_BF16 = 2 } cswap_dtype;

/* Format parameters written into every container header.
 * frame_elems F: > 0, multiple of 1024 (default 4194304).  csr_row C: divides F (default 1024).
 * lz4_block B: multiple of 1024, <= 65536 (default 65536). */
typedef struct {
  uint64_t frame_elems;
  uint32_t csr_row;
  uint32_t lz4_block;
} cswap_format;

/* Sparsity-probe counts: over up to 1024 windows of 256
 * elements (the whole tensor when n <= 2^18). */
typedef struct {
  uint64_t zeros, zero_runs, boundaries, samples, pairs;
} cswap_probe_result;

/* Cost-model calibration (Table II; time model §IV-C).
 * Link: t = alpha + bytes / bw per direction (seconds, bytes/s).
 * beta[codec-1][dir][band][i]: t = b0 + b1*S + b2*S*s, dir 0 = compress, 1 = decompress,
 * bands [0,.2) [.2,.35) [.35,.5) [.5,.65) [.65,.8) [.8,1] of the probed sparsity s, S = raw bytes.
 * LZ4 size model: w*nnz + gamma1*zero_runs + gamma2*w*zeros/255.
 * mode 0 = pipelined (frames overlap codec and copy; margin m), 1 = paper (Eq. 2, m = 0).
 * group_bytes: container bytes per swap-in pipeline step (H2D + decode of whole frames); the
 * pipelined model's swap-in depth G = ceil(K / ceil(group_bytes / frame bytes)), 0 = per frame. */
typedef struct {
  double alpha_d2h, bw_d2h, alpha_h2d, bw_h2d;
  double beta[4][2][6][3];
  double lz4_gamma1, lz4_gamma2;
  double margin;
  int32_t mode;
  int32_t reserved;
  uint64_t frame_elems; /* F used to predict sizes and pipeline depth */
  uint32_t csr_row, lz4_block;
  double group_bytes;   /* swap-in pipeline step (default 32 MiB) */
} cswap_calib;

/* Output of the selector: codec (CSWAP_CODEC_NONE or 1..4), predicted T(c*) and T' (s),
 * per-codec predicted swap time, container bytes, compress and decompress time. */
typedef struct {
  int32_t codec;
  int32_t reserved;
  double t_pred, t_prime;
  double t_codec[4];
  double size[4];
  double t_c[4], t_dc[4];
} cswap_decision;

typedef struct cswap_handle cswap_handle; /* opaque, library-owned swap record */

/* ---- lifecycle ---------------------------------------------------------------------------- */
/* Bind the library to `device` (one device per process), create its internal streams, scratch
 * and pools, and install built-in calibration defaults.  Idempotent for the same device. */
cswap_status cswap_init(int device);
/* Release every resource.  Outstanding handles become invalid. */
cswap_status cswap_shutdown(void);
cswap_status cswap_set_calibration(const cswap_calib* calib);
cswap_status cswap_get_calibration(cswap_calib* out);
/* Default format used by cswap_swap_out and by calls passing fmt = NULL. */
cswap_status cswap_set_format(const cswap_format* fmt);
cswap_status cswap_get_format(cswap_format* out);
/* Launch configuration of the persistent ZVC compress kernel (the knob PAPER.md §IV-D / Alg. 1,
 * :170-214, tunes by Bayesian optimisation on V100: grid x block).  grid = CTAs (0 = automatic:
 * SM count x resident CTAs per SM; clamped to that co-resident maximum, which the kernel's
 * cross-CTA offset protocol needs for forward progress); variant = stage/tile geometry
 * (0: 3 x 32 KiB stages, 8 consumer warps, 2 CTAs/SM; 1: 6 x 16 KiB, 2: 5 x 16 KiB,
 * 3: 4 x 16 KiB; 4: 6 x 32 KiB, 16 consumer warps, 1 CTA/SM; 5: 5 x 32 KiB, 16 warps;
 * 6: 4 x 32 KiB, 16 warps; 7: 3 x 16 KiB, 4 consumer warps, 4 CTAs/SM; 8: 4 x 16 KiB,
 * 4 warps, 3 CTAs/SM; 9: 4 x 24 KiB, 8 consumer warps, 2 CTAs/SM; -1 = default / the
 * CSWAP_ZVC_CFG environment variable).
 * Process-wide; returns CSWAP_ERR_INVALID for a variant outside -1..9. */
cswap_status cswap_set_zvc_launch(uint32_t grid, int32_t variant);

/* ---- device codecs (a3-a10) ------------------------------------------------------------------ */
/* Worst-case container bytes for n elements (0 on invalid arguments).  fmt may be NULL. */
uint64_t cswap_max_compressed_size(uint64_t n, cswap_dtype dtype, cswap_codec codec, const cswap_format* fmt);

/* Compress n elements at d_in (device) into a container at `out` (device or host-mapped pinned
 * memory, out_cap bytes >= cswap_max_compressed_size).  Stream-ordered on `stream`; the container
 * byte count is stored to *out_size (device-visible memory, valid once `stream` reaches it).
 * codec must be NONE/ZVC/RLE/CSR/LZ4.  d_in is only read. */
cswap_status cswap_compress(const void* d_in, uint64_t n, cswap_dtype dtype, cswap_codec codec,
                            const cswap_format* fmt, void* out, uint64_t out_cap, uint64_t* out_size,
                            void* stream);

/* Decompress the container at `in` (device memory, in_size bytes) into n elements at d_out.
 * The header is validated on the device: codec, dtype, n and fmt must agree with it.
 * `err` (device-visible u32, must be 0 on entry; NULL = library word read by
 * cswap_check_device_error) receives CSWAP_ERR_CORRUPT if validation fails on the device; in
 * that case d_out's content is unspecified but no out-of-bounds access happens. */
cswap_status cswap_decompress(const void* in, uint64_t in_size, void* d_out, uint64_t n, cswap_dtype dtype,
                              cswap_codec codec, const cswap_format* fmt, uint32_t* err, void* stream);

/* Synchronise `stream` and return CSWAP_ERR_CORRUPT if a decompress that used err = NULL
 * reported a problem (the word is then cleared). */
cswap_status cswap_check_device_error(void* stream);

/* ---- probe + selector (a1, a2) ----------------------------------------------------------------- */
/* Probe d_in on `stream` and wait for the counts (host result). */
cswap_status cswap_probe(const void* d_in, uint64_t n, cswap_dtype dtype, cswap_probe_result* out, void* stream);
/* Pure host function: Eq. 1-4 with the installed (calib = NULL) or given calibration. */
cswap_status cswap_select_from_probe(uint64_t n, cswap_dtype dtype, const cswap_probe_result* probe,
                                     double hidden_f, double hidden_b, const cswap_calib* calib,
                                     cswap_decision* out);
/* cswap_probe + cswap_select_from_probe with the installed calibration. */
cswap_status cswap_select(const void* d_in, uint64_t n, cswap_dtype dtype, double hidden_f, double hidden_b,
                          void* stream, cswap_decision* out);

/* ---- swap pipeline (a11, a12) --------------------------------------------------------------- */
/* Swap d_in out to library-owned pinned host memory (or the cswap_set_swap_target device),
 * compressed with `codec` (AUTO: probe + selector with the given hidden times, PAPER.md:139
 * Hidden_f/Hidden_b).  Work is ordered after everything already queued on `stream`.
 * Asynchronous: with a fixed codec the call only enqueues the codec kernels on `stream` and hands
 * the copies to the library's executor thread (frames are copied D2H as the kernels publish
 * them) -- it never waits for the device.  AUTO first waits
 * for the probe's counts (the selector runs on the host).
 * Lifetime of d_in: for a compressing codec d_in is read only by kernels on `stream`, so work
 * queued on `stream` afterwards may overwrite it; for CSWAP_CODEC_NONE (raw copy on the library's
 * copy stream) d_in must stay unmodified until cswap_handle_wait() returns or a stream has waited
 * through cswap_handle_record_out(). */
cswap_status cswap_swap_out(const void* d_in, uint64_t n, cswap_dtype dtype, cswap_codec codec, double hidden_f,
                            double hidden_b, void* stream, cswap_handle** out);
/* Restore the tensor into d_out (n elements, device), ordered on `stream`: kernels queued on
 * `stream` afterwards see the restored data.  Waits (on the host) only until the swap-out's
 * copies have been issued; the H2D copies are ordered after the D2H on the device.  The handle
 * keeps its host copy (swap-in may be repeated) until cswap_handle_free. */
cswap_status cswap_swap_in(cswap_handle* h, void* d_out, void* stream);
/* Block until every swap operation on h finished (D2H, and H2D + decode if swap-in was issued);
 * returns deferred asynchronous errors (CORRUPT for a container that failed validation). */
cswap_status cswap_handle_wait(cswap_handle* h);
/* Make `stream` wait (device-side) until h's swap-out finished (d_in reusable). */
cswap_status cswap_handle_record_out(cswap_handle* h, void* stream);
/* codec and decision are known when cswap_swap_out returns (pass NULL for the rest to avoid any
 * wait); container_bytes / host_container wait until the swap-out's copies are issued (the host
 * bytes are complete once cswap_handle_wait returns).  host_container is NULL for a device target. */
cswap_status cswap_handle_query(const cswap_handle* h, cswap_codec* codec, uint64_t* container_bytes,
                                const void** host_container, cswap_decision* decision);
void cswap_handle_free(cswap_handle* h);

/* ---- swap target (NEXT-4b: peer HBM over NVLink, beyond the paper) ---------------------------- */
/* Where cswap_swap_out puts containers from now on: -1 = pinned host memory (default; the paper's
 * target); otherwise a CUDA device -- the device given to cswap_init (a
 * container in local HBM) or a peer reachable by peer-to-peer access (NVLink 5 / NVSwitch on B200).
 * With a device target the codec kernels store the container straight into that device's memory
 * (peer-mapped stores, no host staging and no copy engine); swap-in decompresses straight from it.
 * Containers of a device target have no host copy (cswap_handle_query's host_container = NULL;
 * cswap_handle_copy_container reads them).  The selector keeps using the installed calibration:
 * install one fitted for the peer link (cswap_set_calibration) when AUTO is used.
 * Returns CSWAP_ERR_UNSUPPORTED if `device` cannot be reached by peer access, CSWAP_ERR_INVALID if
 * it does not exist.  Handles already issued keep their own target. */
cswap_status cswap_set_swap_target(int device);
cswap_status cswap_get_swap_target(int* device);
/* Copy h's container (container_bytes of cswap_handle_query, after its swap-out completed) into
 * dst (host or device memory of at least `cap` bytes), ordered on `stream` and synchronised
 * before returning.  Works for every target. */
cswap_status cswap_handle_copy_container(cswap_handle* h, void* dst, uint64_t cap, void* stream);

/* Give cached memory back (like torch.cuda.empty_cache): trims the library's device staging pool
 * to `keep_bytes` (cudaMemPoolTrimTo; the pool otherwise keeps up to CSWAP_POOL_KEEP_MB, default
 * 16 GiB, so that steady swapping never re-maps memory) and unpins host chunks that hold no live
 * container.  Synchronises the device first. */
cswap_status cswap_release_cached(uint64_t keep_bytes);

/* ---- calibration (a13) ----------------------------------------------------------------------- */
/* Ordinary least squares t = b0 + b1*S + b2*S*s over m samples ("linear
 * regression"); beta_out[3].  Returns CSWAP_ERR_INVALID if m < 3 or the design is singular. */
cswap_status cswap_fit_time_model(const double* S, const double* s, const double* t, uint64_t m, double* beta_out);
/* Ordinary least squares t = alpha + bytes / bw (link model); alpha_out, bw_out. */
cswap_status cswap_fit_link(const double* bytes, const double* t, uint64_t m, double* alpha_out, double* bw_out);

/* Generic ordinary least squares y = X beta, X row-major m x p (p <= 8); beta_out[p]. */
cswap_status cswap_fit_linear(const double* X, const double* y, uint64_t m, uint32_t p, double* beta_out);

/* ---- kernel timing (bench / profiling) --------------------------------------------------------- */
/* One record per timed codec launch group: direction 0 = compress, 1 = decompress, 2 = probe;
 * raw_bytes = uncompressed bytes covered, comp_bytes = container bytes read or written (0 if
 * unknown), ms = CUDA-event time on the launch stream; device_ms = %globaltimer difference
 * between two 1-thread stamp kernels placed first and last in the group's graph (the group's
 * own device duration, without the event records' waits behind concurrent PCIe traffic;
 * 0 if unavailable); kernel_ms = the persistent ZVC compress kernel's own %globaltimer span,
 * from CTA 0's start to the last CTA's finish before any host-memory store (0 for other groups;
 * such a group has no stamp kernels, so its device_ms is 0). */
typedef struct {
  int32_t codec, direction;
  uint64_t raw_bytes, comp_bytes;
  double ms;
  double device_ms;
  double kernel_ms;
} cswap_kernel_record;
/* When enabled, the swap pipeline brackets its probe / compress / decompress launches with CUDA
 * events on the stream they are launched on. */
cswap_status cswap_set_kernel_timing(int enable);
/* Wait for pending timing events, copy up to `cap` records into `out`, clear; returns the count. */
uint64_t cswap_collect_kernel_timing(cswap_kernel_record* out, uint64_t cap);

/* ---- diagnostics ---------------------------------------------------------------------------- */
const char* cswap_status_string(cswap_status s);
const char* cswap_last_error(void);
/* Number of kernels this library launched since init (for bench accounting). */
uint64_t cswap_kernel_launches(void);
/* Launch groups (the kernels of one compress, one decompress, one swap-in frame group) run as
 * CUDA graphs: captured on a per-thread stream and replayed on the caller's stream, the
 * executable graph cached per (thread, stream, group kind) and updated in place.  Reason: while a
 * copy engine streams over PCIe, a plainly launched kernel boundary costs 5-10 us on B200, a
 * boundary inside a graph 0.5 us.  Environment CSWAP_GRAPHS=0 launches plainly.
 * Writes the number of graph launches and of instantiations since init (either pointer may be
 * NULL). */
void cswap_graph_stats(uint64_t* launches, uint64_t* instantiations);

#ifdef __cplusplus
}
#endif
#endif /* CSWAP_H */
