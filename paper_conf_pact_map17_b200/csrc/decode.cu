// decode.cu -- inverse of the encoder (R1, R5, R9): one warp per chunk.
//
// Per flag-byte group the eight token headers are read by lanes 0..7 in
// parallel (token j starts at ip + j + 2*popc(flags below j)), their output
// positions come from an 8-lane prefix sum of the token lengths, literals are
// written in parallel, then matches are expanded in order, each by the whole
// warp: out[o + k] = out[o - d + (k mod d)] only reads bytes before o, which are
// final, so overlapping matches (d < l) need no byte-serial loop.  The chunk is
// rebuilt in shared memory and written out with 16-byte stores.  Malformed
// streams set *err = min(1 + chunk index) (err pre-set to 0x7F7F7F7F, fixed up
// to 0 afterwards when no chunk was corrupt).
#include "lzr_internal.cuh"

namespace lzr {

namespace {

constexpr int kDecWarpsMax = 8;
constexpr int32_t kNoError = 0x7F7F7F7F;

__device__ int32_t g_scratch_err;

__global__ void __launch_bounds__(32 * kDecWarpsMax) lzr_decode_kernel(
    const uint8_t* __restrict__ comp, const uint32_t* __restrict__ sizes,
    const uint64_t* __restrict__ offsets, size_t n_bytes, uint32_t C, uint32_t m,
    uint8_t* __restrict__ out, int32_t* err, size_t N, uint32_t buf_stride) {
  extern __shared__ __align__(16) uint8_t dsm[];
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  uint8_t* buf = dsm + (size_t)warp * buf_stride;
  const size_t gw = (size_t)blockIdx.x * (blockDim.x >> 5) + warp;
  const size_t nw = (size_t)gridDim.x * (blockDim.x >> 5);
  for (size_t c = gw; c < N; c += nw) {
    const size_t lo = c * C;
    const uint32_t n = (uint32_t)min((size_t)C, n_bytes - lo);
    const uint32_t S = sizes[c];
    const uint8_t* s = comp + offsets[c];
    uint8_t* dst = out + lo;
    if (S == n) {  // stored raw
      for (uint32_t i = lane; i < n; i += 32) dst[i] = s[i];
      continue;
    }
    bool bad = S > n;
    uint32_t ip = 0, op = 0;
    while (!bad && op < n) {
      if (ip >= S) {
        bad = true;
        break;
      }
      const uint32_t f = s[ip];
      ip += 1;
      const uint32_t j = lane & 7u;
      const uint32_t ism = (f >> j) & 1u;
      const uint32_t toff = ip + j + 2u * __popc(f & ((1u << j) - 1u));
      const uint32_t tsz = 1u + 2u * ism;
      const uint32_t b0 = toff < S ? s[toff] : 0u;
      uint32_t b1 = 0, b2 = 0;
      if (ism) {
        b1 = toff + 1 < S ? s[toff + 1] : 0u;
        b2 = toff + 2 < S ? s[toff + 2] : 0u;
      }
      const uint32_t tlen = ism ? b2 + m : 1u;
      const uint32_t d = (b0 | (b1 << 8)) + 1u;
      uint32_t incl = tlen;
#pragma unroll
      for (int o = 1; o < 8; o <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, incl, o, 8);
        if ((int)j >= o) incl += t;
      }
      const uint32_t ob = op + incl - tlen;  // output position of token j
      const bool reached = ob < n;
      bool e = false;
      if (reached) {
        if (toff + tsz > S) e = true;
        if (ism && (d > ob || ob + tlen > n)) e = true;
      } else if (ism) {
        e = true;  // padding flag bits must be zero
      }
      if (__ballot_sync(kFull, lane < 8 && e)) {
        bad = true;
        break;
      }
      const uint32_t rmask = __ballot_sync(kFull, lane < 8 && reached);
      const uint32_t nt = __popc(rmask);
      const uint32_t fr = f & rmask;
      if (lane < 8 && reached && !ism) buf[ob] = (uint8_t)b0;
      __syncwarp();
      uint32_t mm = fr;
      while (mm) {
        const int jj = __ffs(mm) - 1;
        mm &= mm - 1;
        const uint32_t o = __shfl_sync(kFull, ob, jj);
        const uint32_t dd = __shfl_sync(kFull, d, jj);
        const uint32_t ll = __shfl_sync(kFull, tlen, jj);
        if (dd >= ll) {
          for (uint32_t k = lane; k < ll; k += 32) buf[o + k] = buf[o - dd + k];
        } else {
          for (uint32_t k = lane; k < ll; k += 32) buf[o + k] = buf[o - dd + (k % dd)];
        }
        __syncwarp();
      }
      op += __shfl_sync(kFull, incl, nt - 1);
      ip += nt + 2u * __popc(fr);
    }
    if (!bad && ip != S) bad = true;
    if (bad) {
      if (lane == 0) atomicMin(err, (int32_t)(c + 1));
      continue;
    }
    // write the chunk out: 16-byte stores where aligned, bytes for the tail
    const uint32_t n16 = ((uintptr_t)dst & 15u) ? 0u : (n & ~15u);
    for (uint32_t i = lane * 16; i < n16; i += 32 * 16)
      *reinterpret_cast<uint4*>(dst + i) = *reinterpret_cast<const uint4*>(buf + i);
    for (uint32_t i = n16 + lane; i < n; i += 32) dst[i] = buf[i];
    __syncwarp();
  }
}

__global__ void lzr_decode_fixup_kernel(int32_t* err) {
  if (*err == kNoError) *err = 0;
}

}  // namespace

cudaError_t launch_decode(const uint8_t* comp, const uint32_t* sizes, const uint64_t* offsets,
                          size_t n_bytes, uint32_t C, uint32_t m, uint8_t* out, int32_t* err,
                          int sm_count, int smem_optin, cudaStream_t s, int* launches) {
  const size_t N = (n_bytes + C - 1) / C;
  if (N == 0) {
    if (err) return cudaMemsetAsync(err, 0, sizeof(int32_t), s);
    return cudaSuccess;
  }
  const uint32_t stride = align_up(C + 16, 16);
  int warps = smem_optin / (int)stride;
  if (warps > kDecWarpsMax) warps = kDecWarpsMax;
  if (warps < 1) return cudaErrorInvalidConfiguration;
  const size_t smem = (size_t)warps * stride;
  cudaError_t e = cudaFuncSetAttribute(lzr_decode_kernel,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int32_t* errp = err;
  if (errp) {
    e = cudaMemsetAsync(errp, 0x7F, sizeof(int32_t), s);
    if (e != cudaSuccess) return e;
  }
  // a private error word is needed when the caller passes none
  if (!errp) {
    e = cudaGetSymbolAddress((void**)&errp, g_scratch_err);
    if (e != cudaSuccess) return e;
  }
  size_t blocks = (N + warps - 1) / warps;
  const size_t cap = (size_t)sm_count * 4;
  if (blocks > cap) blocks = cap;
  lzr_decode_kernel<<<(unsigned)blocks, warps * 32, smem, s>>>(comp, sizes, offsets, n_bytes, C, m,
                                                              out, errp, N, stride);
  if (launches) ++*launches;
  e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  if (err) {
    lzr_decode_fixup_kernel<<<1, 1, 0, s>>>(err);
    if (launches) ++*launches;
    e = cudaGetLastError();
  }
  return e;
}

}  // namespace lzr
