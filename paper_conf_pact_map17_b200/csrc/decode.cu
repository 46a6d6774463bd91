// decode.cu -- inverse of the encoder (R1, R5, R9): one warp per chunk.
//
// The chunk's compressed stream is first staged into shared memory with
// aligned 4-byte loads (one coalesced pass), so every later header/token read
// is a shared-memory access.  Per flag-byte group, lanes 0..7 read the eight
// token headers in parallel (token j starts at ip + j + 2*popc(flags below j)),
// an 8-lane prefix sum of token lengths gives their output positions, literals
// are written in parallel, then matches are expanded in order, each by the
// whole warp: out[o + k] = out[o - d + (k mod d)] only reads bytes before o,
// which are final, so overlapping matches (d < l) need no byte-serial loop.
// The chunk is rebuilt in shared memory and written out with 16-byte stores;
// raw chunks are copied with 16-byte stores from funnel-shifted 4-byte loads.
// Malformed streams set *err = min(1 + chunk index) (err pre-set to 0x7F7F7F7F,
// fixed up to 0 afterwards when no chunk was corrupt).
#include "lzr_internal.cuh"

namespace lzr {

namespace {

constexpr int kDecWarpsMax = 8;
constexpr int32_t kNoError = 0x7F7F7F7F;

__device__ int32_t g_scratch_err;

// Word i of the aligned view of src - mis, reading only bytes in [mis, mis + len)
// (edge words byte by byte, so no access leaves the caller's buffer).
__device__ __forceinline__ uint32_t load_word(const uint8_t* src, uint32_t mis, uint32_t len,
                                              uint32_t i) {
  const uint32_t b = i << 2;
  if (b >= mis && b + 4 <= mis + len) return __ldg(reinterpret_cast<const uint32_t*>(src - mis) + i);
  uint32_t v = 0;
  for (uint32_t t = 0; t < 4; ++t) {
    const uint32_t x = b + t;
    if (x >= mis && x < mis + len) v |= (uint32_t)src[x - mis] << (8 * t);
  }
  return v;
}

// Stage src[0..S) (arbitrary alignment) into smem: buf + (src & 3) holds src[0].
__device__ __forceinline__ const uint8_t* stage_stream(uint8_t* buf, const uint8_t* src, uint32_t S,
                                                       uint32_t lane) {
  const uint32_t mis = (uint32_t)((uintptr_t)src & 3u);
  uint32_t* b32 = reinterpret_cast<uint32_t*>(buf);
  const uint32_t words = (mis + S + 3) >> 2;
  for (uint32_t i = lane; i < words; i += 32) b32[i] = load_word(src, mis, S, i);
  return buf + mis;
}

__global__ void __launch_bounds__(32 * kDecWarpsMax, 1) lzr_decode_kernel(
    const uint8_t* __restrict__ comp, const uint32_t* __restrict__ sizes,
    const uint64_t* __restrict__ offsets, size_t n_bytes, uint32_t C, uint32_t m,
    uint8_t* __restrict__ out, int32_t* err, size_t N, uint32_t buf_stride) {
  extern __shared__ __align__(16) uint8_t dsm[];
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  uint8_t* obuf = dsm + (size_t)warp * buf_stride;  // rebuilt chunk (C bytes)
  uint8_t* sbuf = obuf + align_up(C, 16);           // staged stream (C + 4 bytes)
  const size_t gw = (size_t)blockIdx.x * (blockDim.x >> 5) + warp;
  const size_t nw = (size_t)gridDim.x * (blockDim.x >> 5);
  for (size_t c = gw; c < N; c += nw) {
    const size_t lo = c * C;
    const uint32_t n = (uint32_t)min((size_t)C, n_bytes - lo);
    const uint32_t S = sizes[c];
    const uint8_t* src = comp + offsets[c];
    uint8_t* dst = out + lo;
    if (S == n) {  // stored raw: funnel-shifted 4-byte loads -> 16-byte stores
      const uint32_t mis = (uint32_t)((uintptr_t)src & 3u);
      const uint32_t n16 = ((uintptr_t)dst & 15u) ? 0u : (n & ~15u);
      for (uint32_t i = lane * 16; i < n16; i += 32 * 16) {
        const uint32_t w0 = (mis + i) >> 2;
        uint32_t v[5];
#pragma unroll
        for (int t = 0; t < 5; ++t) v[t] = load_word(src, mis, n, w0 + t);
        const uint32_t sh = mis << 3;
        *reinterpret_cast<uint4*>(dst + i) =
            make_uint4(__funnelshift_r(v[0], v[1], sh), __funnelshift_r(v[1], v[2], sh),
                       __funnelshift_r(v[2], v[3], sh), __funnelshift_r(v[3], v[4], sh));
      }
      for (uint32_t i = n16 + lane; i < n; i += 32) dst[i] = src[i];
      continue;
    }
    bool bad = S > n;
    const uint8_t* s = bad ? sbuf : stage_stream(sbuf, src, S, lane);
    __syncwarp();
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
      if (lane < 8 && reached && !ism) obuf[ob] = (uint8_t)b0;
      __syncwarp();
      uint32_t mm = fr;
      while (mm) {
        const int jj = __ffs(mm) - 1;
        mm &= mm - 1;
        const uint32_t o = __shfl_sync(kFull, ob, jj);
        const uint32_t dd = __shfl_sync(kFull, d, jj);
        const uint32_t ll = __shfl_sync(kFull, tlen, jj);
        if (dd >= ll) {
          for (uint32_t k = lane; k < ll; k += 32) obuf[o + k] = obuf[o - dd + k];
        } else {
          for (uint32_t k = lane; k < ll; k += 32) obuf[o + k] = obuf[o - dd + (k % dd)];
        }
        __syncwarp();
      }
      op += __shfl_sync(kFull, incl, nt - 1);
      ip += nt + 2u * __popc(fr);
    }
    if (!bad && ip != S) bad = true;
    if (bad) {
      if (lane == 0) atomicMin(err, (int32_t)(c + 1));
      __syncwarp();
      continue;
    }
    // write the chunk out: 16-byte stores where aligned, bytes for the tail
    const uint32_t n16 = ((uintptr_t)dst & 15u) ? 0u : (n & ~15u);
    for (uint32_t i = lane * 16; i < n16; i += 32 * 16)
      *reinterpret_cast<uint4*>(dst + i) = *reinterpret_cast<const uint4*>(obuf + i);
    for (uint32_t i = n16 + lane; i < n; i += 32) dst[i] = obuf[i];
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
  const uint32_t stride = align_up(C, 16) + align_up(C + 8, 16);  // rebuilt chunk + staged stream
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
  // as many CTAs as fit (shared memory bound), at most one wave of chunks
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lzr_decode_kernel, warps * 32, smem);
  if (e != cudaSuccess || per_sm < 1) per_sm = 1;
  size_t blocks = (N + warps - 1) / warps;
  const size_t cap = (size_t)sm_count * per_sm;
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
