// decode.cu -- inverse of the encoder (R1, R5, R9): one warp per chunk, 32
// tokens (four flag-byte groups) per step.
//
// The four flag bytes of a step are a short dependent chain (group g + 1
// starts 9 + 2 popc(f_g) bytes after group g); then lane t owns token t: its
// stream offset is ip_g + 1 + j + 2 popc(f_g below j), its output position a
// 32-lane prefix sum of token lengths.  A step's stream bytes come from a
// 128-byte window held one word per lane (loaded coalesced while the previous
// step copies, bytes outside [src, src + S) read as 0) by shuffle.  The chunk
// is rebuilt in shared memory: literals of the step are stored in parallel,
// then the step's matches are resolved in rounds -- a match whose source bytes
// lie below the first unresolved match's output (or that is the first one) is
// final-sourced, so all such matches copy at once: short ones one lane each,
// byte-serially (which also gives overlapping matches, d < l, their R5
// meaning), long ones by the whole warp (out[o + k] = out[o - d + (k mod d)]
// only reads bytes before o).  The chunk is written out with 16-byte stores;
// raw chunks are copied with 16-byte stores from funnel-shifted 4-byte loads.
// Malformed streams set *err = min(1 + chunk index) (err pre-set to 0x7F7F7F7F,
// fixed up to 0 afterwards when no chunk was corrupt); with err == NULL nothing
// is reported (include/lzr.h) and the library keeps no global error word.
// (An output-parallel variant -- each step's output rebuilt in 32-byte windows,
// lane = byte, token found by a REDUX.OR of the window's token starts, sources
// by (o - ob) mod d and in-window pointer jumping, stream staged in shared
// memory -- measured no faster: text 230-248 vs 243 GB/s, zero-runs 318-395 vs
// 677.)
#include <mutex>

#include "lzr_internal.cuh"

namespace lzr {

namespace {

// CTA shape of the decode grid (see launch_decode): 2 warps, and enough
// resident CTAs per SM that registers do not cut occupancy below ~48 warps
#ifndef LZR_DEC_WARPS
#define LZR_DEC_WARPS 2
#endif
#ifndef LZR_DEC_MINB
#define LZR_DEC_MINB 24
#endif
constexpr int32_t kNoError = 0x7F7F7F7F;
// (1 x B200, 256 MiB, mix/text GB/s: 8 -> 347/208, 12 -> 392/241, 16 ->
// 402/248, 24 -> 404/250; byte-serial copies 4 at a time with d >= 4: 389/234)
#ifndef LZR_DEC_LANE_MAX
#define LZR_DEC_LANE_MAX 16
#endif
constexpr uint32_t kLaneCopyMax = LZR_DEC_LANE_MAX;  // matches up to this length: one lane, byte-serial
// (measured and not kept, 1 x B200, 256 MiB, output GB/s mix/text/zero-runs:
// an L1 prefetch of the stream's lines at chunk start 356/247/702 vs
// 386/247/667; short matches copied 4 source bytes per step from two aligned
// words 383/238/694)

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


// CF, MF != 0: specialised for chunk size CF and min match MF (compile-time)
template <uint32_t CF, uint32_t MF>
__global__ void __launch_bounds__(32 * LZR_DEC_WARPS, LZR_DEC_MINB) lzr_decode_kernel(
    const uint8_t* __restrict__ comp, const uint32_t* __restrict__ sizes,
    const uint64_t* __restrict__ offsets, size_t n_bytes, uint32_t C_in, uint32_t m_in,
    uint8_t* __restrict__ out, int32_t* err, size_t N, uint32_t buf_stride_in, uint64_t err_base) {
  const uint32_t C = CF ? CF : C_in, m = MF ? MF : m_in;
  const uint32_t buf_stride = CF ? align_up(CF, 16) : buf_stride_in;
  extern __shared__ __align__(16) uint8_t dsm[];
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  uint8_t* obuf = dsm + (size_t)warp * buf_stride;  // rebuilt chunk (C bytes)
  const size_t gw = (size_t)blockIdx.x * (blockDim.x >> 5) + warp;
  const size_t nw = (size_t)gridDim.x * (blockDim.x >> 5);
  const uint32_t g = lane >> 3, j = lane & 7u;
  const uint32_t below = (1u << j) - 1u;
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
    // A step reads at most 4 groups (<= 100 bytes) from ip.  The 128 stream
    // bytes from ip (32 aligned words, one per lane: a coalesced load, bytes
    // outside the stream read as 0) are loaded before the step -- the next
    // step's window is issued as soon as this step's end is known, so its
    // latency hides under the match copies -- and the parse takes its bytes
    // from the window by shuffle instead of a chain of dependent loads.
    const uint32_t mis = (uint32_t)((uintptr_t)src & 3u);
    uint32_t ip = 0, op = 0;
    uint32_t wbase = mis >> 2;  // first word of the window (aligned view src - mis)
    uint32_t win = bad ? 0u : load_word(src, mis, S, wbase + lane);
    while (!bad && op < n) {
      const uint32_t wb = wbase, wv = win;
      auto sb = [&](uint32_t x) -> uint32_t {  // stream byte x (x <= ip + 101), 0 past the end
        const uint32_t xx = x + mis;
        return (__shfl_sync(kFull, wv, (xx >> 2) - wb) >> ((xx & 3u) << 3)) & 0xFFu;
      };
      // the four groups of this step: flag byte and stream offset
      uint32_t f = 0, ipg = 0;
      {
        uint32_t x = ip;
#pragma unroll
        for (uint32_t t = 0; t < 4; ++t) {
          const uint32_t ft = sb(x);
          if (t == g) {
            f = ft;
            ipg = x;
          }
          x += 9u + 2u * __popc(ft);
        }
      }
      const uint32_t ism = (f >> j) & 1u;
      const uint32_t toff = ipg + 1u + j + 2u * __popc(f & below);
      const uint32_t tsz = 1u + 2u * ism;
      // the token's 3 header bytes from the two window words around toff
      uint32_t b0, b1, b2;
      {
        const uint32_t xx = toff + mis;
        const uint32_t wi = (xx >> 2) - wb;
        const uint32_t lo = __shfl_sync(kFull, wv, wi), hi = __shfl_sync(kFull, wv, wi + 1);
        const uint32_t v = __funnelshift_r(lo, hi, (xx & 3u) << 3);
        b0 = v & 0xFFu;
        b1 = ism ? (v >> 8) & 0xFFu : 0u;
        b2 = ism ? (v >> 16) & 0xFFu : 0u;
      }
      const uint32_t tlen = ism ? b2 + m : 1u;
      const uint32_t d = (b0 | (b1 << 8)) + 1u;
      uint32_t incl = tlen;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, incl, o);
        if ((int)lane >= o) incl += t;
      }
      const uint32_t ob = op + incl - tlen;  // output position of token `lane`
      // a group is live when the groups before it did not finish the chunk
      const uint32_t gstart = __shfl_sync(kFull, ob, lane & ~7u);
      const bool live = gstart < n;
      const bool reached = live && ob < n;
      bool e = false;
      if (live && ipg >= S) e = true;  // flag byte past the stream
      if (reached) {
        if (toff + tsz > S) e = true;
        if (ism && (d > ob || ob + tlen > n)) e = true;
      } else if (live && ism) {
        e = true;  // padding flag bits must be zero
      }
      if (__any_sync(kFull, e)) {
        bad = true;
        break;
      }
      const uint32_t rmask = __ballot_sync(kFull, reached);  // a prefix of the lanes
      const uint32_t last = 31u - __clz(rmask);
      {  // the next step's window, issued now
        const uint32_t ipn = __shfl_sync(kFull, toff + tsz, last);
        wbase = (ipn + mis) >> 2;
        win = ipn < S ? load_word(src, mis, S, wbase + lane) : 0u;
      }
      if (reached && !ism) obuf[ob] = (uint8_t)b0;
      __syncwarp();
      uint32_t pend = __ballot_sync(kFull, reached && ism);
      // bytes a match needs before its own output (the rest overlaps itself)
      const uint32_t need_end = ob - d + min(tlen, d);
      while (pend) {
        const uint32_t f0 = (uint32_t)(__ffs(pend) - 1);
        const uint32_t first_ob = __shfl_sync(kFull, ob, f0);
        const bool mine = (pend >> lane) & 1u;
        const uint32_t ready = __ballot_sync(kFull, mine && (lane == f0 || need_end <= first_ob));
        const bool go = (ready >> lane) & 1u;
        if (go && tlen <= kLaneCopyMax) {
          for (uint32_t k = 0; k < tlen; ++k) obuf[ob + k] = obuf[ob - d + k];
        }
        uint32_t lng = ready & __ballot_sync(kFull, tlen > kLaneCopyMax);
        while (lng) {
          const int jj = __ffs(lng) - 1;
          lng &= lng - 1;
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
        __syncwarp();
        pend &= ~ready;
      }
      op = __shfl_sync(kFull, ob + tlen, last);
      ip = __shfl_sync(kFull, toff + tsz, last);
    }
    if (!bad && ip != S) bad = true;
    if (bad) {
      if (lane == 0 && err) atomicMin(err, (int32_t)(c + 1 + err_base));
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

cudaError_t decode_err_init(int32_t* err, cudaStream_t s) {
  return cudaMemsetAsync(err, 0x7F, sizeof(int32_t), s);
}

cudaError_t decode_err_fini(int32_t* err, cudaStream_t s, int* launches) {
  lzr_decode_fixup_kernel<<<1, 1, 0, s>>>(err);
  if (launches) ++*launches;
  return cudaGetLastError();
}

cudaError_t launch_decode(const uint8_t* comp, const uint32_t* sizes, const uint64_t* offsets,
                          size_t n_bytes, uint32_t C, uint32_t m, uint8_t* out, int32_t* err,
                          int sm_count, int smem_optin, cudaStream_t s, int* launches,
                          uint64_t err_base, bool err_own) {
  const size_t N = (n_bytes + C - 1) / C;
  if (N == 0) {
    if (err && err_own) return cudaMemsetAsync(err, 0, sizeof(int32_t), s);
    return cudaSuccess;
  }
  const uint32_t stride = align_up(C, 16);  // rebuilt chunk
// Grid: 2 warps (chunks) per CTA and one CTA per 2 chunks, so the hardware
// block scheduler balances chunks of very different cost (raw copies vs text)
// as CTAs retire; a persistent one-wave grid of 16-warp CTAs left SMs idle at
// the end (1 x B200, 256 MiB, output GB/s mix/text/zero-runs: 16-warp one-wave
// 290/214/596; full grids of 16/8/4/2/1-warp CTAs 302/309/347/380/369 mix,
// text 239-242 except 211 at 1 warp (32 CTAs per SM = 32 warps))
#ifndef LZR_DEC_ONEWAVE
#define LZR_DEC_ONEWAVE 0
#endif
  int warps = smem_optin / (int)stride;
  if (warps > LZR_DEC_WARPS) warps = LZR_DEC_WARPS;
  if (C > 16384) warps = 1;  // one chunk per CTA: more CTAs fit an SM
  if (warps < 1) return cudaErrorInvalidConfiguration;
  const size_t smem = (size_t)warps * stride;
  // The dynamic shared-memory limit is raised once per device to the opt-in
  // maximum (never lowered, so concurrent callers with different chunk sizes
  // cannot undercut each other); the occupancy is cached per smem size.
  struct Cached {
    bool attr;
    size_t smem;
    int per_sm;
  };
  static Cached cache[64] = {};
  static std::mutex mu;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  int per_sm = 0;
  {
    std::lock_guard<std::mutex> lk(mu);
    if (!cache[dev].attr) {
      e = cudaFuncSetAttribute(lzr_decode_kernel<0, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin);
      if (e == cudaSuccess)
        e = cudaFuncSetAttribute(lzr_decode_kernel<4096, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin);
      if (e != cudaSuccess) return e;
      cache[dev].attr = true;
    }
    if (cache[dev].smem == smem) per_sm = cache[dev].per_sm;
  }
  if (per_sm == 0) {
    // (LZR_DEC_ONEWAVE: at most one resident wave of CTAs, warps loop over chunks)
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lzr_decode_kernel<0, 0>, warps * 32, smem);
    if (e != cudaSuccess || per_sm < 1) per_sm = 1;
    std::lock_guard<std::mutex> lk(mu);
    cache[dev].smem = smem;
    cache[dev].per_sm = per_sm;
  }
  int32_t* errp = err;
  if (errp && err_own) {
    e = decode_err_init(errp, s);
    if (e != cudaSuccess) return e;
  }
  size_t blocks = (N + warps - 1) / warps;
  const size_t cap = (size_t)sm_count * per_sm;
  if (LZR_DEC_ONEWAVE && blocks > cap) blocks = cap;
  if (C == 4096 && m == 4)  // the configs' chunk size and min match
    lzr_decode_kernel<4096, 4><<<(unsigned)blocks, warps * 32, smem, s>>>(comp, sizes, offsets, n_bytes, C, m,
                                                                         out, errp, N, stride, err_base);
  else
  lzr_decode_kernel<0, 0><<<(unsigned)blocks, warps * 32, smem, s>>>(comp, sizes, offsets, n_bytes, C, m,
                                                              out, errp, N, stride, err_base);
  if (launches) ++*launches;
  e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  if (err && err_own) e = decode_err_fini(err, s, launches);
  return e;
}

}  // namespace lzr
