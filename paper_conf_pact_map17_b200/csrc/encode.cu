// encode.cu -- the compression hot path on sm_100a: one warp per chunk.
//
// Steps (§3.2(2) "The GPU allocates multiple
// threads for each chunk. Each stage performs its own LZ compression algorithm
// with its own history buffer and look-ahead buffer."):
//   a2  stage the chunk (= its whole history window, R2) into shared memory with
//       a 1-D bulk TMA copy (cp.async.bulk + mbarrier);
//   a3  longest-match search.  Exact candidates are the earlier positions with
//       the same first k = min(m,4) bytes (any match of length >= m >= k starts
//       with them).  The warp counting-sorts positions by a hash of that key
//       into buckets that stay in ascending position order, so the candidates of
//       p are a contiguous run of slots below p's own slot, nearest first.  The
//       32 lanes evaluate 32 candidates at a time; each candidate's capped
//       common-prefix length is packed as (len << 16 | 0xFFFF - (d - 1)) and
//       reduced with REDUX.MAX, which selects "longest, then nearest" (R6, R7).
//       A candidate beyond the best length so far must also match the byte at
//       that length (a necessary condition for being strictly longer), so most
//       farther candidates cost one compare.  Search stops at the cap (exact:
//       nothing beats the cap) or when the bucket / window is exhausted.
//   a4  greedy selection (R8): the warp walks p = 0 .. n-1.  A 1-bit-per-position
//       "has a same-key candidate inside the window" bitmap lets it emit runs of
//       up to 32 literals per step (ballot-free: one funnel shift of the bitmap).
//   a5  flag-byte LZSS encoding (R1) straight into the chunk's workspace slot,
//       raw fallback when the stream would not be shorter than the chunk (R9).
// The serial result is reproduced exactly: the best match at p depends only on
// (chunk bytes, p, W, m, M), not on the parse.
#include "lzr_internal.cuh"

namespace lzr {

namespace {

constexpr int kMaxWarps = 16;

__device__ __forceinline__ uint32_t khash(uint32_t key, uint32_t hbits) {
  return (key * 0x9E3779B1u) >> (32 - hbits);
}

// Capped common-prefix length of data[a..] and data[b..] (a > b allowed to
// overlap: compares original bytes, = byte-serial copy semantics, R5).
__device__ __forceinline__ uint32_t lcp_words(const uint8_t* d, uint32_t a, uint32_t b,
                                              uint32_t maxlen) {
  uint32_t l = 0;
  while (l < maxlen) {
    uint32_t x = ld32u(d, a + l) ^ ld32u(d, b + l);
    if (x) {
      l += (uint32_t)(__ffs(x) - 1) >> 3;
      return l < maxlen ? l : maxlen;
    }
    l += 4;
  }
  return maxlen;
}

struct EncState {
  uint32_t opos, fpos, cnt, fbits;
};

// Emit L (1..32) literal tokens x[p..p+L) (R1: literal = 1 byte, flag bit 0).
__device__ __forceinline__ void emit_literals(uint8_t* out, const uint8_t* data, uint32_t p,
                                              uint32_t L, uint32_t n, EncState& e,
                                              uint32_t lane) {
  const uint32_t c0 = e.cnt;
  if (lane < L) {
    uint32_t t = c0 + lane;
    uint32_t nf = (c0 == 0) ? (lane >> 3) + 1 : (t >> 3);  // flag bytes opened up to this token
    uint32_t pos = e.opos + lane + nf;
    if (pos < n) out[pos] = data[p + lane];
    // a group opened and completed inside this run holds only literals: flag 0
    if ((t & 7u) == 0 && lane + 7 < L && pos - 1 < n) out[pos - 1] = 0;
  }
  // the group open before this run is completed inside it: its flag byte is final
  if (c0 != 0 && c0 + L >= 8 && lane == 0 && e.fpos < n) out[e.fpos] = (uint8_t)e.fbits;
  const uint32_t nf_tot = (c0 == 0) ? ((L - 1) >> 3) + 1 : ((c0 + L - 1) >> 3);
  const uint32_t cend = (c0 + L) & 7u;
  if (!(c0 != 0 && c0 + L < 8) && cend != 0) {
    // a new group opened inside this run stays open
    uint32_t ts = (c0 + L - 1) & ~7u;
    uint32_t is = ts - c0;
    uint32_t nfs = (c0 == 0) ? (is >> 3) + 1 : (ts >> 3);
    e.fpos = e.opos + is + nfs - 1;
    e.fbits = 0;
  }
  e.opos += L + nf_tot;
  e.cnt = cend;
}

// Emit one match token (R1: 3 bytes (d-1) u16 LE, (l-m) u8; flag bit 1).
__device__ __forceinline__ void emit_match(uint8_t* out, uint32_t d, uint32_t l, uint32_t m,
                                           uint32_t n, EncState& e, uint32_t lane) {
  if (e.cnt == 0) {
    e.fpos = e.opos;
    e.opos += 1;
    e.fbits = 0;
  }
  if (lane == 0) {
    uint32_t o = e.opos;
    if (o < n) out[o] = (uint8_t)((d - 1) & 0xFF);
    if (o + 1 < n) out[o + 1] = (uint8_t)((d - 1) >> 8);
    if (o + 2 < n) out[o + 2] = (uint8_t)(l - m);
  }
  e.fbits |= 1u << e.cnt;
  e.opos += 3;
  e.cnt += 1;
  if (e.cnt == 8) {
    if (lane == 0 && e.fpos < n) out[e.fpos] = (uint8_t)e.fbits;
    e.cnt = 0;
  }
}

// Longest, then nearest, capped match at p (a3).  Returns the packed key
// (len << 16) | (0xFFFF - (d-1)), or 0 when no candidate reaches m.
__device__ __forceinline__ uint32_t best_match(const uint8_t* data, const uint16_t* sorted,
                                               const uint16_t* slot, uint32_t p, uint32_t n,
                                               const EncArgs& a, uint32_t lane) {
  const uint32_t kp = ld32u(data, p) & a.kmask;
  const uint32_t hp = khash(kp, a.L.hbits);
  const uint32_t cap = min(a.M, n - p);  // p < n - m + 1  =>  cap >= m >= k
  uint32_t best = 0, blen = 0;
  for (int sb = (int)slot[p] - 1; sb >= 0; sb -= 32) {
    const int s = sb - (int)lane;
    uint32_t q = 0;
    bool stop = true, cand = false;
    if (s >= 0) {
      q = sorted[s];
      const uint32_t kq = ld32u(data, q) & a.kmask;
      const bool in_window = p - q <= a.W;
      stop = !in_window || (kq != kp && khash(kq, a.L.hbits) != hp);
      cand = !stop && kq == kp;
    }
    const uint32_t stopmask = __ballot_sync(kFull, stop);
    const uint32_t first_stop = stopmask ? (uint32_t)(__ffs(stopmask) - 1) : 32u;
    uint32_t pk = 0;
    if (cand && lane < first_stop) {
      // strictly longer than blen requires a match at offset blen (blen < cap here)
      if (blen == 0 || data[q + blen] == data[p + blen]) {
        const uint32_t l = a.kbytes + lcp_words(data, p + a.kbytes, q + a.kbytes, cap - a.kbytes);
        if (l >= a.m) pk = (l << 16) | (0xFFFFu - (p - q - 1));
      }
    }
    best = max(best, __reduce_max_sync(kFull, pk));
    blen = best >> 16;
    if (blen >= cap || first_stop < 32) break;
  }
  return best;
}

// Build the per-chunk candidate structure (sorted buckets, slots, bitmap).
__device__ __forceinline__ void build_index(const uint8_t* data, uint16_t* sorted, uint16_t* slot,
                                            uint32_t* bm, uint32_t n, uint32_t P, const EncArgs& a,
                                            uint32_t lane) {
  const uint32_t hb = a.L.hbits;
  const uint32_t B = 1u << hb;
  uint32_t* hist = reinterpret_cast<uint32_t*>(slot);  // B u16 counters, two per word
  for (uint32_t i = lane; i < B / 2; i += 32) hist[i] = 0;
  __syncwarp();
  // histogram of bucket sizes
  for (uint32_t p = lane; p < P; p += 32) {
    const uint32_t h = khash(ld32u(data, p) & a.kmask, hb);
    atomicAdd(&hist[h >> 1], 1u << ((h & 1u) << 4));
  }
  __syncwarp();
  // exclusive scan of the B u16 counters, 64 per round
  uint32_t carry = 0;
  for (uint32_t w0 = 0; w0 < B / 2; w0 += 32) {
    const bool act = w0 + lane < B / 2;
    const uint32_t wv = act ? hist[w0 + lane] : 0;
    const uint32_t c0 = wv & 0xFFFFu, sum = c0 + (wv >> 16);
    uint32_t incl = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(kFull, incl, o);
      if ((int)lane >= o) incl += t;
    }
    const uint32_t excl = incl - sum + carry;
    if (act) hist[w0 + lane] = (excl & 0xFFFFu) | ((excl + c0) << 16);
    carry += __shfl_sync(kFull, incl, 31);
  }
  __syncwarp();
  // stable scatter: positions in ascending order within each bucket
  uint16_t* cur = slot;
  const uint32_t lt = lanemask_lt();
  for (uint32_t p0 = 0; p0 < P; p0 += 32) {
    const uint32_t p = p0 + lane;
    const bool act = p < P;
    const uint32_t h = act ? khash(ld32u(data, p) & a.kmask, hb) : 0xFFFFFFFFu;
    const uint32_t peers = __match_any_sync(kFull, h);
    const uint32_t rank = __popc(peers & lt);
    const uint32_t basev = act ? cur[h] : 0;
    if (act) sorted[basev + rank] = (uint16_t)p;
    __syncwarp();
    if (act && lane == 31u - __clz(peers)) cur[h] = (uint16_t)(basev + __popc(peers));
    __syncwarp();
  }
  // slot of each position (the bucket cursors are dead now)
  for (uint32_t s = lane; s < P; s += 32) slot[sorted[s]] = (uint16_t)s;
  __syncwarp();
  // bitmap: p has a same-key earlier position inside the window
  for (uint32_t w = 0; w < a.L.bm_words; ++w) {
    const uint32_t p = w * 32 + lane;
    bool has = false;
    if (p < P) {
      const uint32_t kp = ld32u(data, p) & a.kmask;
      const uint32_t hp = khash(kp, hb);
      for (int s = (int)slot[p] - 1; s >= 0; --s) {
        const uint32_t q = sorted[s];
        const uint32_t kq = ld32u(data, q) & a.kmask;
        if (kq == kp) {
          has = p - q <= a.W;  // nearest same-key position decides
          break;
        }
        if (khash(kq, hb) != hp) break;
      }
    }
    const uint32_t b = __ballot_sync(kFull, has);
    if (lane == 0) bm[w] = b;
  }
  __syncwarp();
}

__global__ void __launch_bounds__(32 * kMaxWarps, 1) lzr_encode_kernel(const EncArgs a) {
  extern __shared__ __align__(128) uint8_t smem[];
  const uint32_t lane = threadIdx.x & 31u;
  const uint32_t warp = threadIdx.x >> 5;
  uint8_t* base = smem + (size_t)warp * a.L.per_warp;
  uint8_t* data = base;
  uint16_t* sorted = reinterpret_cast<uint16_t*>(base + a.L.off_sorted);
  uint16_t* slot = reinterpret_cast<uint16_t*>(base + a.L.off_slot);
  uint32_t* bm = reinterpret_cast<uint32_t*>(base + a.L.off_bm);
  uint64_t* bar = reinterpret_cast<uint64_t*>(base + a.L.off_mbar);

  if (lane == 0) {
    mbar_init(bar, 1);
    fence_mbar_init();
  }
  __syncwarp();
  uint32_t phase = 0;

  for (;;) {
    uint32_t c = 0;
    if (lane == 0) c = atomicAdd(a.counter, 1u);
    c = __shfl_sync(kFull, c, 0);
    if (c >= a.N) break;
    const size_t lo = (size_t)c * a.C;
    const uint32_t n = (uint32_t)min((size_t)a.C, a.n_bytes - lo);
    const uint8_t* src = a.in + lo;

    // ---- a2: stage the chunk (TMA bulk for the 16-byte multiple, LDG for the tail)
    fence_proxy_async_smem();  // prior generic accesses to `data` before the async write
    __syncwarp();
    const uint32_t n16 = n & ~15u;
    if (lane == 0 && n16) {
      mbar_arrive_expect_tx(bar, n16);
      tma_bulk_g2s(data, src, n16, bar);
    }
    for (uint32_t i = n16 + lane; i < n; i += 32) data[i] = src[i];
    for (uint32_t i = n + lane; i < align_up(n, 16) + 16; i += 32) data[i] = 0;
    if (n16) {
      mbar_wait_parity(bar, phase);
      phase ^= 1u;
    }
    __syncwarp();

    // ---- a3 index
    const uint32_t P = n >= a.m ? n - a.m + 1 : 0;  // positions that can start a match
    build_index(data, sorted, slot, bm, n, P, a, lane);

    // ---- a3/a4/a5: greedy walk + encode
    uint8_t* out = a.slots + lo;
    EncState e{0, 0, 0, 0};
    bool raw = false;
    uint32_t p = 0;
    while (p < n) {
      uint32_t bits = 0;
      if (p < P) bits = __funnelshift_r(bm[p >> 5], bm[(p >> 5) + 1], p & 31u);
      if (bits == 0) {
        const uint32_t L = min(32u, n - p);
        emit_literals(out, data, p, L, n, e, lane);
        p += L;
      } else {
        const uint32_t f = (uint32_t)(__ffs(bits) - 1);
        if (f) {
          emit_literals(out, data, p, f, n, e, lane);
          p += f;
        } else {
          const uint32_t r = best_match(data, sorted, slot, p, n, a, lane);
          const uint32_t l = r >> 16;
          if (l >= a.m) {
            emit_match(out, 0xFFFFu - (r & 0xFFFFu) + 1, l, a.m, n, e, lane);
            p += l;
          } else {
            emit_literals(out, data, p, 1, n, e, lane);
            p += 1;
          }
        }
      }
      if (e.opos >= n) {
        raw = true;  // stream not shorter than the chunk: stored raw (R9)
        break;
      }
    }
    if (!raw && e.cnt != 0 && lane == 0) out[e.fpos] = (uint8_t)e.fbits;
    if (lane == 0) a.sizes[c] = raw ? n : e.opos;
    __syncwarp();
  }
}

}  // namespace

cudaError_t launch_encode(const EncArgs& a, int sm_count, int smem_optin, cudaStream_t s,
                          int* launches) {
  int warps = smem_optin / (int)a.L.per_warp;
  if (warps > kMaxWarps) warps = kMaxWarps;
  if (warps < 1) return cudaErrorInvalidConfiguration;
  const size_t smem = (size_t)warps * a.L.per_warp;
  cudaError_t err = cudaFuncSetAttribute(lzr_encode_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err != cudaSuccess) return err;
  const uint32_t need = (a.N + warps - 1) / warps;
  const uint32_t grid = need < (uint32_t)sm_count ? need : (uint32_t)sm_count;
  lzr_encode_kernel<<<grid, warps * 32, smem, s>>>(a);
  if (launches) ++*launches;
  return cudaGetLastError();
}

}  // namespace lzr
