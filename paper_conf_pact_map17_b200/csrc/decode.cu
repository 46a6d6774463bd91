// decode.cu -- inverse of the encoder (R1, R5, R9): one warp per chunk, 32
// tokens (four flag-byte groups) per step.
//
// Parse: the four flag bytes of a step are a short dependent chain (group g + 1
// starts 9 + 2 popc(f_g) bytes after group g; the lanes of group g stop after
// g hops); then lane t owns token t: its stream offset is ip_g + 1 + j +
// 2 popc(f_g below j), its output position a 32-lane prefix sum of token
// lengths.  A step's stream bytes come from a 128-byte window held one word per
// lane (loaded coalesced while the previous step copies, bytes outside
// [src, src + S) read as 0) by shuffle.
// Output: the chunk is rebuilt in shared memory.  Literals are stored by their
// lanes.  Matches whose source bytes all lie below the step's start (and that
// do not overlap themselves) are "final-sourced": they are listed in token
// order and copied by all 32 lanes at once, each match by 32/P lanes (P = their
// count rounded up to a power of two), so a step's short copies cost about
// l/(32/P) iterations instead of max(l).  The rest -- long matches, matches
// that read this step's output, overlapping ones (d < l, R5) -- follow in token
// order, each by the whole warp (overlapping: out[o + k] = out[o - d + k mod
// d], all below o).  The chunk is written out with 16-byte stores; raw chunks
// are copied with 16-byte stores from funnel-shifted 4-byte loads.
// Malformed streams set *err = min(1 + chunk index) (err pre-set to 0x7F7F7F7F,
// fixed up to 0 afterwards when no chunk was corrupt); with err == NULL nothing
// is reported (include/lzr.h) and the library keeps no global error word.
// (Replaced and measured: round 1-2's lane-per-match byte-serial
// copies in dependency rounds -- 23% of the text decode's instructions in the
// byte loop; output-parallel 32-byte windows, lane = byte, token by an
// OR-reduction of the window's token starts -- as costly per byte.)
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
constexpr uint32_t kCopyList = 32 * sizeof(uint2);  // per warp, after its chunk buffer
// final-sourced matches up to this length go to the lane-spread copy (1 x
// B200, 256 MiB, output GB/s mix/text/zero-runs: 16 -> 562/362/871, 32 ->
// 568/367/875, 64 -> 566/366/871; the copy list packs the length in 8 bits)
#ifndef LZR_DEC_LANE_MAX
#define LZR_DEC_LANE_MAX 32
#endif
constexpr uint32_t kLaneCopyMax = LZR_DEC_LANE_MAX;
static_assert(kLaneCopyMax < 256, "copy-list length field");
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


// shared-memory bytes by 32-bit address (keeps the rebuilt chunk's base in one
// register; ordered, the copies below rely on program order within a lane)
__device__ __forceinline__ uint32_t lds8(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts8(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

// byte (x & 3) of w in all four bytes
__device__ __forceinline__ uint32_t prmt_rc8(uint32_t w, uint32_t x) {
  uint32_t r;
  asm("prmt.b32.rc8 %0, %1, 0, %2;" : "=r"(r) : "r"(w), "r"(x));
  return r;
}

// inclusive prefix sum over the warp (shfl.up's own predicate marks lanes >= delta)
__device__ __forceinline__ uint32_t warp_incl_sum(uint32_t v) {
#pragma unroll
  for (uint32_t o = 1; o < 32; o <<= 1)
    asm("{\n\t.reg .u32 t;\n\t.reg .pred p;\n\tshfl.sync.up.b32 t|p, %0, %1, 0, -1;\n\t@p add.u32 %0, %0, t;\n\t}"
        : "+r"(v) : "r"(o));
  return v;
}

// CF, MF != 0: specialised for chunk size CF and min match MF (compile-time)
template <uint32_t CF, uint32_t MF>
__global__ void __launch_bounds__(32 * LZR_DEC_WARPS, LZR_DEC_MINB) lzr_decode_kernel(
    const uint8_t* __restrict__ comp, const uint32_t* __restrict__ sizes,
    const uint64_t* __restrict__ offsets, size_t n_bytes, uint32_t C_in, uint32_t m_in,
    uint8_t* __restrict__ out, int32_t* err, size_t N, uint32_t buf_stride_in, uint64_t err_base) {
  const uint32_t C = CF ? CF : C_in, m = MF ? MF : m_in;
  const uint32_t buf_stride = CF ? align_up(CF, 16) + kCopyList : buf_stride_in;
  extern __shared__ __align__(16) uint8_t dsm[];
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  uint8_t* obuf = dsm + (size_t)warp * buf_stride;  // rebuilt chunk (C bytes)
  // the step's final-sourced matches (source, destination | length << 24)
  uint2* clist = reinterpret_cast<uint2*>(obuf + buf_stride - kCopyList);
  const size_t gw = (size_t)blockIdx.x * (blockDim.x >> 5) + warp;
  const size_t nw = (size_t)gridDim.x * (blockDim.x >> 5);
  const uint32_t g = lane >> 3, j = lane & 7u;
  const uint32_t below = (1u << j) - 1u, jbit = 1u << j;  // token j's flag bit and the ones before it
  const uint32_t sbuf = smem_u32(obuf);
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
    // Stream positions below are in the aligned view src - mis ("x"
    // coordinates: stream byte i is x = i + mis).  A step reads at most 4
    // groups (<= 100 bytes) from ip: the 128 bytes from ip's word (one aligned
    // word per lane, a coalesced load, bytes outside the stream read as 0) are
    // loaded before the step -- the next step's window is issued as soon as
    // this step's end is known, so its latency hides under the copies -- and
    // the parse takes its bytes from the window by shuffle.
    const uint32_t mis = (uint32_t)((uintptr_t)src & 3u);
    const uint32_t Sx = S + mis;
    uint32_t ip = mis, op = 0;
    uint32_t wbase = 0;  // first word of the window
    uint32_t win = bad ? 0u : load_word(src, mis, S, lane);
    while (!bad && op < n) {
      const uint32_t wb = wbase, wv = win;
      // stream byte at x (x <= ip + 100) replicated into all four bytes of
      // the result (prmt.rc8 takes the byte index from x's low bits):
      // popc(rep) = 4 popc(byte), and rep & mask = byte & mask for masks < 256
      auto sbyte4 = [&](uint32_t x) -> uint32_t {
        return prmt_rc8(__shfl_sync(kFull, wv, (x >> 2) - wb), x);
      };
      // the flag-byte chain: the lanes of group g stop after g hops
      uint32_t x = ip;
#pragma unroll
      for (uint32_t t = 0; t < 3; ++t) {
        const uint32_t ft = sbyte4(x);
        if (g > t) x += 9u + (__popc(ft) >> 1);
      }
      const uint32_t f = sbyte4(x);
      const bool ism = (f & jbit) != 0u;
      const uint32_t toff = x + 1u + j + 2u * __popc(f & below);
      const uint32_t tend = toff + (ism ? 3u : 1u);  // stream position after the token
      // the token's 3 header bytes from the two window words around toff
      uint32_t hv;
      {
        const uint32_t wi = (toff >> 2) - wb;
        hv = __funnelshift_r(__shfl_sync(kFull, wv, wi), __shfl_sync(kFull, wv, wi + 1), (toff & 3u) << 3);
      }
      const uint32_t tlen = ism ? __byte_perm(hv, 0u, 0x4442u) + m : 1u;
      const uint32_t d = (hv & 0xFFFFu) + 1u;
      const uint32_t incl = warp_incl_sum(tlen);
      const uint32_t ob = op + incl - tlen;  // output position of token `lane`
      // a group is live when the groups before it did not finish the chunk;
      // a token is reached when it starts below n (ob grows with the lane)
      const bool reached = ob < n;
      const uint32_t rmask = __ballot_sync(kFull, reached);  // a prefix of the lanes
      const bool live = (rmask >> (lane & ~7u)) & 1u;
      // R15: flag byte or token past the stream, d beyond the output, a match
      // past n or a set padding flag bit (ob >= n => ob + tlen > n)
      const bool e = live && (x >= Sx || (ism && (d > ob || ob + tlen > n)) || (reached && tend > Sx));
      if (__any_sync(kFull, e)) {
        bad = true;
        break;
      }
      const uint32_t last = 31u - __clz(rmask);
      const uint32_t ipn = __shfl_sync(kFull, tend, last);
      const uint32_t opn = __shfl_sync(kFull, ob + tlen, last);
      {  // the next step's window, issued now
        wbase = ipn >> 2;
        win = ipn < Sx ? load_word(src, mis, S, wbase + lane) : 0u;
      }
      // Output.  Literals are stored by their lanes.  A match whose source
      // bytes all lie below op (the step's start; overlapping ones d < l only
      // need [ob - d, ob)) is final-sourced: the short ones copy at once, one
      // lane each, byte-serially.  The rest -- long matches and matches that
      // read this step's output -- follow in token order, each by the whole
      // warp.
      if (reached && !ism) sts8(sbuf + ob, hv & 0xFFu);
      const bool rdy = reached && ism && tlen <= kLaneCopyMax && d >= tlen && ob - d + tlen <= op;
      if (reached && !ism) sts8(sbuf + ob, hv & 0xFFu);
      const uint32_t rset = __ballot_sync(kFull, rdy);
      if (rset) {
        // the nr final-sourced matches are listed in token order; lane L
        // copies bytes h, h + H, ... of match L mod P (P = nr rounded up to
        // a power of two, h = L / P, H = 32 / P): no byte of them is read by
        // another (d >= l, sources below op)
        if (rdy) clist[__popc(rset & lanemask_lt())] = make_uint2(sbuf + ob - d, (sbuf + ob) | (tlen << 24));
        __syncwarp();
        const uint32_t nr = __popc(rset), lg = 32u - __clz(nr - 1u);
        const uint32_t mi = lane & ((1u << lg) - 1u);
        if (mi < nr) {
          const uint2 cl = clist[mi];
          const uint32_t len = cl.y >> 24, da = cl.y & 0xFFFFFFu, step = 32u >> lg;
          for (uint32_t k = lane >> lg; k < len; k += step) sts8(da + k, lds8(cl.x + k));
        }
      }
      uint32_t rest = __ballot_sync(kFull, reached && ism && !rdy);
      __syncwarp();
      while (rest) {
        const uint32_t jj = __ffs(rest) - 1u;
        rest &= rest - 1u;
        const uint32_t o = __shfl_sync(kFull, ob, jj);
        const uint32_t dd = __shfl_sync(kFull, d, jj);
        const uint32_t ll = __shfl_sync(kFull, tlen, jj);
        if (dd >= 32u || dd >= ll) {  // a window of 32 never reads its own bytes
          for (uint32_t k0 = 0; k0 < ll; k0 += 32u) {  // (warp-uniform trip count: the barrier below)
            const uint32_t k = k0 + lane;
            if (k < ll) sts8(sbuf + o + k, lds8(sbuf + o - dd + k));
            __syncwarp();
          }
        } else {  // d < 32, overlapping: out[o + k] = out[o - d + k mod d], all below o
          const uint32_t sb = sbuf + o - dd, adv = 32u % dd;
          uint32_t r = lane % dd;
          for (uint32_t k = lane; k < ll; k += 32u) {
            sts8(sbuf + o + k, lds8(sb + r));
            r += adv;
            if (r >= dd) r -= dd;
          }
          __syncwarp();
        }
      }
      op = opn;
      ip = ipn;
    }
    if (!bad && ip != Sx) bad = true;
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
  const uint32_t stride = align_up(C, 16) + kCopyList;  // rebuilt chunk + copy list
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
