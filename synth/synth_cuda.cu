/* synth/synth_cuda.cu -- device side of the seeded generator (see synth_core.h).
 * One thread per chunk; the same syn_fill_chunk() as the host build. */
#include <cuda_runtime.h>

#include "synth_core.h"

__global__ void syn_fill_kernel(uint8_t* out, size_t n, uint32_t C, int cls, uint64_t seed,
                                uint64_t first, size_t N, const syn_tables* t) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= N) return;
  size_t b = i * C;
  uint32_t ni = (uint32_t)(n - b < C ? n - b : C);
  syn_fill_chunk(out + b, ni, cls, seed, first + i, t);
}

extern "C" int syn_fill_device(void* d_out, size_t n, uint32_t chunk_size, int cls,
                               uint64_t seed, uint64_t first_chunk, const void* d_tables,
                               cudaStream_t stream) {
  if (chunk_size == 0 || cls < 0 || (cls & ~SYN_DEDUP) >= SYN_NCLASS || (n && (!d_out || !d_tables))) return -1;
  size_t N = (n + chunk_size - 1) / chunk_size;
  if (N == 0) return 0;
  unsigned threads = 128;
  unsigned blocks = (unsigned)((N + threads - 1) / threads);
  syn_fill_kernel<<<blocks, threads, 0, stream>>>((uint8_t*)d_out, n, chunk_size, cls, seed,
                                                  first_chunk, N, (const syn_tables*)d_tables);
  return cudaGetLastError() == cudaSuccess ? 0 : -4;
}
