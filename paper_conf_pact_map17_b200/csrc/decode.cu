// decode.cu -- inverse of the encoder (R1, R5, R9): one warp per chunk, up to
// 64 tokens (eight flag-byte groups) per step.
//
// Parse: a step's stream bytes come from a 128-byte window held one word per
// lane (loaded coalesced while the previous step copies, bytes outside
// [src, src + S) read as 0) by shuffle; the step takes the groups that lie
// wholly inside it (text: all eight, most steps).  The flag bytes are a short
// dependent chain (group g + 1 starts 9 + 2 popc(f_g) bytes after group g; the
// lanes of group g stop after g hops); lane L owns tokens j0 = 2 (L mod 4) and
// j0 + 1 of group L / 4: stream offset ip_g + 1 + j0 + 2 popc(f_g below j0),
// output position a 32-lane prefix sum of the lanes' two token lengths.
// Output: the chunk is rebuilt in shared memory.  Literals are stored by their
// lanes.  Matches whose source bytes all lie below the step's start (and that
// do not overlap themselves) are "final-sourced": the first 32 of a step are
// listed in token order (shared memory) and copied by all 32 lanes at once,
// each match by 32/P lanes (P = their count rounded up to a power of two), so
// a step's short copies cost about l/(32/P) iterations instead of max(l).  The rest -- long matches, matches
// that read this step's output, overlapping ones (d < l, R5) -- follow in token
// order, each by the whole warp (overlapping: out[o + k] = out[o - d + k mod
// d], all below o).  The chunk is written out with 16-byte stores; raw chunks
// are copied with 16-byte stores from funnel-shifted 4-byte loads.
// Schedule: given a workspace, the chunks are decoded costliest first (raw
// last, compressed ones by size; a bucket sort of the sizes, below), so the
// end of the grid runs short chunks and a CTA's two chunks cost about the same.
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
  if (b + 4 <= mis || b >= mis + len) return 0u;
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

// Debug build (-DLZR_DEC_CHECK, tools/check_decode.sh): every shared-memory
// access of the rebuild traps unless it stays inside the chunk's bytes and
// reads only bytes already final (compute-sanitizer is not available on the
// GPU pool; this is the bounds check that replaces it for the decoder).
#ifdef LZR_DEC_CHECK
#define DEC_ASSERT(c) \
  do {            \
    if (!(c)) __trap(); \
  } while (0)
#else
#define DEC_ASSERT(c) \
  do {            \
  } while (0)
#endif

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
    uint8_t* __restrict__ out, int32_t* err, size_t N, uint32_t buf_stride_in, uint64_t err_base,
    const uint32_t* __restrict__ perm) {
  const uint32_t C = CF ? CF : C_in, m = MF ? MF : m_in;
  const uint32_t buf_stride = CF ? align_up(CF, 16) + kCopyList : buf_stride_in;
  extern __shared__ __align__(16) uint8_t dsm[];
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  uint8_t* obuf = dsm + (size_t)warp * buf_stride;  // rebuilt chunk (C bytes)
  // the step's final-sourced matches (source, destination | length << 24)
  uint2* clist = reinterpret_cast<uint2*>(obuf + buf_stride - kCopyList);
  const size_t gw = (size_t)blockIdx.x * (blockDim.x >> 5) + warp;
  const size_t nw = (size_t)gridDim.x * (blockDim.x >> 5);
  const uint32_t g = lane >> 2, j0 = (lane & 3u) << 1;  // tokens j0, j0 + 1 of group g
  const uint32_t below0 = (1u << j0) - 1u, bit0 = 1u << j0, bit1 = 2u << j0;
  const uint32_t sbuf = smem_u32(obuf);
  for (size_t ci = gw; ci < N; ci += nw) {
    const size_t c = perm ? (size_t)perm[ci] : ci;  // the schedule: costliest chunks first
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
        if (i >= 4u && i + 20u <= n) {  // the five words lie inside the chunk's bytes
          const uint32_t* sw = reinterpret_cast<const uint32_t*>(src - mis) + w0;
#pragma unroll
          for (int t = 0; t < 5; ++t) v[t] = __ldg(sw + t);
        } else {
#pragma unroll
          for (int t = 0; t < 5; ++t) v[t] = load_word(src, mis, n, w0 + t);
        }
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
    // coordinates: stream byte i is x = i + mis).  A step parses the groups
    // (up to 8, 64 tokens) that lie wholly inside a 128-byte window from ip's
    // word (one aligned word per lane, a coalesced load, bytes outside the
    // stream read as 0); the next step's window is issued as soon as this
    // step's end is known, so its latency hides under the copies.
    const uint32_t mis = (uint32_t)((uintptr_t)src & 3u);
    const uint32_t Sx = S + mis;
    uint32_t ip = mis, op = 0;
    uint32_t wbase = 0;  // first word of the window
    uint32_t win = bad ? 0u : load_word(src, mis, S, lane);
    while (!bad && op < n) {
      const uint32_t wb = wbase, wv = win;
      const uint32_t wend = (wb << 2) + 128u;
      // stream byte at x replicated into all four bytes (prmt.rc8 takes the
      // byte index from x's low bits): popc(rep) = 4 popc(byte), and
      // rep & mask = byte & mask for masks < 256
      auto sbyte4 = [&](uint32_t x) -> uint32_t {
        return prmt_rc8(__shfl_sync(kFull, wv, (x >> 2) - wb), x);
      };
      // the flag-byte chain: the lanes of group g stop after g hops
      uint32_t x = ip;
#pragma unroll
      for (uint32_t t = 0; t < 7; ++t) {
        const uint32_t ft = sbyte4(x);
        if (g > t) x += 9u + (__popc(ft) >> 1);
      }
      const uint32_t f = sbyte4(x);
      // this step takes the groups whose flag byte and 8 token slots lie in
      // the window (a prefix of the groups; group 0 always fits)
      const bool fits = x + 9u + (__popc(f) >> 1) <= wend;
      // tokens 2(lane mod 4) and +1 of group g
      const bool ism0 = fits && (f & bit0) != 0u, ism1 = fits && (f & bit1) != 0u;
      const uint32_t toff0 = x + 1u + j0 + 2u * __popc(f & below0);
      const uint32_t toff1 = toff0 + (ism0 ? 3u : 1u);
      const uint32_t tend0 = toff1, tend1 = toff1 + (ism1 ? 3u : 1u);
      // both tokens' header bytes from the three window words from toff0's
      uint32_t hv0, hv1;
      {
        const uint32_t wi = (toff0 >> 2) - wb;
        const uint32_t w0 = __shfl_sync(kFull, wv, wi), w1 = __shfl_sync(kFull, wv, wi + 1u),
                       w2 = __shfl_sync(kFull, wv, wi + 2u);
        hv0 = __funnelshift_r(w0, w1, (toff0 & 3u) << 3);
        const uint32_t r = toff1 - (toff0 & ~3u);  // 1..6
        hv1 = r < 4u ? __funnelshift_r(w0, w1, r << 3) : __funnelshift_r(w1, w2, (r - 4u) << 3);
      }
      const uint32_t tlen0 = ism0 ? __byte_perm(hv0, 0u, 0x4442u) + m : (fits ? 1u : 0u);
      const uint32_t tlen1 = ism1 ? __byte_perm(hv1, 0u, 0x4442u) + m : (fits ? 1u : 0u);
      const uint32_t d0 = (hv0 & 0xFFFFu) + 1u, d1 = (hv1 & 0xFFFFu) + 1u;
      const uint32_t incl = warp_incl_sum(tlen0 + tlen1);
      const uint32_t ob0 = op + incl - tlen0 - tlen1, ob1 = ob0 + tlen0;  // output positions
      // a token is reached when it is parsed and starts below n; a group is
      // live when its first token is reached
      const bool reached0 = fits && ob0 < n, reached1 = fits && ob1 < n;
      const uint32_t rm0 = __ballot_sync(kFull, reached0), rm1 = __ballot_sync(kFull, reached1);
      const bool live = (rm0 >> (lane & ~3u)) & 1u;
      // R15: flag byte or token past the stream, d beyond the output, a match
      // past n or a set padding flag bit (ob >= n => ob + tlen > n)
      const bool e = live && (x >= Sx || (ism0 && (d0 > ob0 || ob0 + tlen0 > n)) ||
                              (ism1 && (d1 > ob1 || ob1 + tlen1 > n)) || (reached0 && tend0 > Sx) ||
                              (reached1 && tend1 > Sx));
      if (__any_sync(kFull, e)) {
        bad = true;
        break;
      }
      // the last reached token: token 1 of lane l0 if reached, else token 0
      const uint32_t l0 = 31u - __clz(rm0);
      const uint32_t ipn = __shfl_sync(kFull, reached1 ? tend1 : tend0, l0);
      const uint32_t opn = __shfl_sync(kFull, reached1 ? ob1 + tlen1 : ob0 + tlen0, l0);
      {  // the next step's window, issued now
        wbase = ipn >> 2;
        win = ipn < Sx ? load_word(src, mis, S, wbase + lane) : 0u;
      }
      // Output.  Literals are stored by their lanes.  Matches whose source
      // bytes all lie below op and that do not overlap themselves are listed in
      // token order and copied by all lanes at once; the rest follow in token
      // order, each by the whole warp.
      DEC_ASSERT(!(reached0 && !ism0) || ob0 < n);
      DEC_ASSERT(!(reached1 && !ism1) || ob1 < n);
      if (reached0 && !ism0) sts8(sbuf + ob0, hv0 & 0xFFu);
      if (reached1 && !ism1) sts8(sbuf + ob1, hv1 & 0xFFu);
      bool rdy0 = reached0 && ism0 && tlen0 <= kLaneCopyMax && d0 >= tlen0 && ob0 - d0 + tlen0 <= op;
      bool rdy1 = reached1 && ism1 && tlen1 <= kLaneCopyMax && d1 >= tlen1 && ob1 - d1 + tlen1 <= op;
      const uint32_t R0 = __ballot_sync(kFull, rdy0), R1 = __ballot_sync(kFull, rdy1);
      if (R0 | R1) {
        // the list holds 32 entries: later ones go to the token-order pass
        const uint32_t lt = lanemask_lt();
        const uint32_t rk = __popc(R0 & lt) + __popc(R1 & lt);
        rdy0 = rdy0 && rk < 32u;
        rdy1 = rdy1 && rk + rdy0 < 32u;
        if (rdy0) clist[rk] = make_uint2(sbuf + ob0 - d0, (sbuf + ob0) | (tlen0 << 24));
        if (rdy1) clist[rk + rdy0] = make_uint2(sbuf + ob1 - d1, (sbuf + ob1) | (tlen1 << 24));
        __syncwarp();
        const uint32_t nr = min(__popc(R0) + __popc(R1), 32u), lg = 32u - __clz(nr - 1u);
        // lane L copies bytes h, h + H, ... of entry L mod P (P = nr rounded
        // up to a power of two, h = L / P, H = 32 / P)
        const uint32_t mi = lane & ((1u << lg) - 1u);
        if (mi < nr) {
          const uint2 cl = clist[mi];
          const uint32_t len = cl.y >> 24, da = cl.y & 0xFFFFFFu, step = 32u >> lg;
          DEC_ASSERT(cl.x >= sbuf && cl.x + len <= sbuf + op && da >= sbuf + op && da + len <= sbuf + n);
          uint32_t k = lane >> lg;
          for (; k + step < len; k += 2u * step) {  // two bytes per iteration
            const uint32_t b0 = lds8(cl.x + k), b1 = lds8(cl.x + k + step);
            sts8(da + k, b0);
            sts8(da + k + step, b1);
          }
          if (k < len) sts8(da + k, lds8(cl.x + k));
        }
      }
      uint32_t X0 = __ballot_sync(kFull, reached0 && ism0 && !rdy0);
      uint32_t X1 = __ballot_sync(kFull, reached1 && ism1 && !rdy1);
      __syncwarp();
      while (X0 | X1) {
        const uint32_t jj = __ffs(X0 | X1) - 1u;
        const bool second = !((X0 >> jj) & 1u);  // token 1 of lane jj
        if (second) X1 &= X1 - 1u;
        else X0 &= ~(1u << jj);
        const uint32_t o = __shfl_sync(kFull, second ? ob1 : ob0, jj);
        const uint32_t dd = __shfl_sync(kFull, second ? d1 : d0, jj);
        const uint32_t ll = __shfl_sync(kFull, second ? tlen1 : tlen0, jj);
        if (ll <= 32u && dd >= ll) {  // one window, no loop (most of them)
          DEC_ASSERT(lane >= ll || (dd <= o && o + lane < n));
          if (lane < ll) sts8(sbuf + o + lane, lds8(sbuf + o - dd + lane));
          __syncwarp();
        } else if (dd >= 32u || dd >= ll) {  // a window of 32 never reads its own bytes
          for (uint32_t k0 = 0; k0 < ll; k0 += 32u) {  // (warp-uniform trip count: the barrier below)
            const uint32_t k = k0 + lane;
            DEC_ASSERT(k >= ll || (dd <= o && o + k < n));
            if (k < ll) sts8(sbuf + o + k, lds8(sbuf + o - dd + k));
            __syncwarp();
          }
        } else {  // d < 32, overlapping: out[o + k] = out[o - d + k mod d], all below o
          // lane mod d and 32 mod d for d < 32 by a float reciprocal: q = floor((x + 0.5) / d)
          // is exact for x <= 32, d < 32 (checked for every pair in IEEE single)
          const float rd = __frcp_rn((float)dd);
          const uint32_t sb = sbuf + o - dd;
          const uint32_t adv = 32u - dd * (uint32_t)(32.5f * rd);
          uint32_t r = lane - dd * (uint32_t)(((float)lane + 0.5f) * rd);
          for (uint32_t k = lane; k < ll; k += 32u) {
            DEC_ASSERT(sb >= sbuf && sb + r < sbuf + o && o + k < n);
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

// ---- the decode schedule: chunks costliest first ------------
// A chunk's decode cost is known from its size: a raw chunk is a copy (the
// cheapest), a compressed one costs about its token count, ~S.  Bucket 0 =
// raw, 1 + min(31, 32 S / C) otherwise; the schedule lists bucket 32 first.
// Taking the long chunks first shortens the end-of-grid tail and puts chunks
// of similar cost into the same CTA (1 x B200, 256 MiB mix with its chunks
// reordered so: 0.429 -> 0.382 ms per decode).
constexpr uint32_t kSchedB = 33;

__device__ __forceinline__ uint32_t sched_bucket(const uint32_t* sizes, size_t c, size_t n_bytes,
                                                 uint32_t C) {
  const uint32_t n = (uint32_t)min((size_t)C, n_bytes - c * C);
  const uint32_t S = sizes[c];
  return S >= n ? 0u : 1u + min(31u, (uint32_t)(((uint64_t)S * 32u) / C));
}

__global__ void lzr_sched_hist_kernel(const uint32_t* __restrict__ sizes, size_t N, size_t n_bytes,
                                      uint32_t C, uint32_t* counts) {
  __shared__ uint32_t h[kSchedB];
  for (uint32_t i = threadIdx.x; i < kSchedB; i += blockDim.x) h[i] = 0;
  __syncthreads();
  for (size_t c = (size_t)blockIdx.x * blockDim.x + threadIdx.x; c < N; c += (size_t)gridDim.x * blockDim.x)
    atomicAdd(&h[sched_bucket(sizes, c, n_bytes, C)], 1u);
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < kSchedB; i += blockDim.x)
    if (h[i]) atomicAdd(&counts[i], h[i]);
}

__global__ void lzr_sched_scatter_kernel(const uint32_t* __restrict__ sizes, size_t N, size_t n_bytes,
                                         uint32_t C, const uint32_t* __restrict__ counts,
                                         uint32_t* cursors, uint32_t* __restrict__ perm) {
  __shared__ uint32_t base[kSchedB];
  if (threadIdx.x == 0) {
    uint32_t acc = 0;
    for (int b = (int)kSchedB - 1; b >= 0; --b) {
      base[b] = acc;
      acc += counts[b];
    }
  }
  __syncthreads();
  const uint32_t lane = threadIdx.x & 31u;
  for (size_t c = (size_t)blockIdx.x * blockDim.x + threadIdx.x; c < N; c += (size_t)gridDim.x * blockDim.x) {
    const uint32_t b = sched_bucket(sizes, c, n_bytes, C);
    // one atomic per bucket per warp
    const uint32_t am = __activemask();
    const uint32_t peers = __match_any_sync(am, b);
    const uint32_t leader = __ffs(peers) - 1u;
    uint32_t off = 0;
    if (lane == leader) off = atomicAdd(&cursors[b], (uint32_t)__popc(peers));
    off = __shfl_sync(peers, off, leader);
    perm[base[b] + off + __popc(peers & lanemask_lt())] = (uint32_t)c;
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
                          uint64_t err_base, bool err_own, uint32_t* sched) {
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
  const uint32_t* perm = nullptr;
  if (sched && N > 1 && N <= 0xFFFFFFFFull) {  // the costliest-first schedule (workspace given)
    uint32_t* counts = sched;
    uint32_t* cursors = sched + 64;
    uint32_t* pm = sched + 128;
    e = cudaMemsetAsync(sched, 0, 128 * sizeof(uint32_t), s);
    if (e != cudaSuccess) return e;
    const unsigned sg = (unsigned)min((N + 255) / 256, (size_t)sm_count * 8);
    lzr_sched_hist_kernel<<<sg, 256, 0, s>>>(sizes, N, n_bytes, C, counts);
    lzr_sched_scatter_kernel<<<sg, 256, 0, s>>>(sizes, N, n_bytes, C, counts, cursors, pm);
    if (launches) *launches += 2;
    perm = pm;
  }
  const size_t cap = (size_t)sm_count * per_sm;
  if (LZR_DEC_ONEWAVE && blocks > cap) blocks = cap;
  if (C == 4096 && m == 4)  // the configs' chunk size and min match
    lzr_decode_kernel<4096, 4><<<(unsigned)blocks, warps * 32, smem, s>>>(comp, sizes, offsets, n_bytes, C, m,
                                                                         out, errp, N, stride, err_base, perm);
  else
  lzr_decode_kernel<0, 0><<<(unsigned)blocks, warps * 32, smem, s>>>(comp, sizes, offsets, n_bytes, C, m,
                                                              out, errp, N, stride, err_base, perm);
  if (launches) ++*launches;
  e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  if (err && err_own) e = decode_err_fini(err, s, launches);
  return e;
}

}  // namespace lzr
