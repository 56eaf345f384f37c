// stubs.cu — temporary: codecs not yet implemented in this build return cudaErrorNotSupported.
#include "kernels.h"
namespace cswap {
uint64_t lz4_scratch_bytes(uint64_t n, int w, uint64_t, uint32_t B) { return (cdiv(n * w, B) + 1) * 65552; }
cudaError_t launch_lz4_compress(const void*, uint64_t, int, uint64_t, uint32_t, uint8_t*, uint64_t*, uint8_t*, const Scratch&, int, cudaStream_t) { return cudaErrorNotSupported; }
cudaError_t launch_lz4_decompress(const uint8_t*, void*, uint64_t, int, uint64_t, uint32_t, uint32_t, uint32_t, const Scratch&, uint32_t*, cudaStream_t) { return cudaErrorNotSupported; }
}
