// kernels.h — internal launchers (not part of the public C ABI; see include/cswap.h).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "common.cuh"

namespace cswap {

// api.cu: records the start event of the pending kernel timer (if timing is enabled) right
// before a launcher's first kernel
void timing_kernel_start(cudaStream_t st);

// container.cu
cudaError_t launch_header_only(uint8_t* out, int codec, int dtype, uint64_t F, uint32_t param, uint64_t* out_size,
                               cudaStream_t st);
cudaError_t launch_prep(const uint8_t* in, uint64_t in_size, int codec, int dtype, uint64_t n, uint64_t F,
                        uint32_t param, const Scratch& sc, uint32_t* err, bool reset_err, cudaStream_t st);
// zero `words` u32 words with a kernel (not the copy engine)
cudaError_t launch_zero_words(void* p, uint64_t words, cudaStream_t st);
// frame_bytes in sc.aux2[k] -> frame table, frame starts in sc.aux[k], header, *out_size
cudaError_t launch_finalize(uint8_t* out, int codec, int dtype, uint64_t n, uint64_t F, uint32_t param,
                            const Scratch& sc, uint64_t* out_size, cudaStream_t st);
cudaError_t launch_err_merge(const uint32_t* src, uint32_t* dst, cudaStream_t st);
// one thread writes %globaltimer (ns) to dst (device-visible; here mapped pinned memory)
cudaError_t launch_stamp(uint64_t* dst, cudaStream_t st, bool first);
cudaError_t launch_none_compress(const void* in, uint64_t n, int w, uint64_t F, int dtype, uint8_t* out,
                                 uint64_t* out_size, cudaStream_t st);
cudaError_t launch_none_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, const Scratch& sc,
                                   uint32_t* err, cudaStream_t st);
// counts3[c] = count << 16 | tag (host-mapped; the host polls for the tag)
cudaError_t launch_probe(const void* in, uint64_t n, int w, uint64_t* counts3, uint32_t tag, const Scratch& sc,
                         uint32_t epoch, cudaStream_t st);
// swap-out progress of a finished compress group: prog[k] = kProgReady | end offset of frame k
cudaError_t launch_publish_frames(const uint8_t* out, uint32_t K, uint64_t* prog, cudaStream_t st);

// zvc.cu
uint32_t zvc_tiles(uint64_t n, int w, uint64_t F, uint32_t k0, uint32_t k1, uint32_t* tpf_out);
void zvc_compress_scratch(uint64_t n, int w, uint64_t F, uint64_t* tiles, uint64_t* aux);
bool zvc_set_launch(uint32_t grid, int variant);  // cswap_set_zvc_launch
cudaError_t launch_zvc_compress(const void* in, uint64_t n, int w, uint64_t F, uint8_t* out, uint64_t* out_size,
                                const Scratch& sc, uint32_t epoch, int dtype, cudaStream_t st);
cudaError_t launch_zvc_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t k0,
                                  uint32_t k1, const Scratch& sc, uint32_t epoch, uint32_t* err, cudaStream_t st);

// rle.cu
uint32_t rle_tiles(uint64_t n, int w, uint64_t F);
cudaError_t launch_rle_compress(const void* in, uint64_t n, int w, uint64_t F, uint8_t* out, uint64_t* out_size,
                                const Scratch& sc, uint32_t epoch, int dtype, cudaStream_t st);
uint64_t rle_decompress_tmp_bytes(uint64_t n, uint64_t F, uint32_t k0, uint32_t k1);
cudaError_t launch_rle_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t k0,
                                  uint32_t k1, const Scratch& sc, uint32_t epoch, uint32_t* err, uint8_t* tmp,
                                  cudaStream_t st);

// csr.cu
cudaError_t launch_csr_compress(const void* in, uint64_t n, int w, uint64_t F, uint32_t C, uint8_t* out,
                                uint64_t* out_size, const Scratch& sc, uint32_t epoch, int dtype, cudaStream_t st);
cudaError_t launch_csr_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t C,
                                  uint32_t k0, uint32_t k1, const Scratch& sc, uint32_t* err, cudaStream_t st);

// lz4.cu
uint64_t lz4_scratch_bytes(uint64_t n, int w, uint64_t F, uint32_t B);
cudaError_t launch_lz4_compress(const void* in, uint64_t n, int w, uint64_t F, uint32_t B, uint8_t* out,
                                uint64_t* out_size, uint8_t* slots, const Scratch& sc, int dtype, cudaStream_t st);
cudaError_t launch_lz4_decompress(const uint8_t* in, void* out, uint64_t n, int w, uint64_t F, uint32_t B,
                                  uint32_t k0, uint32_t k1, const Scratch& sc, uint32_t* err, cudaStream_t st);

}  // namespace cswap
