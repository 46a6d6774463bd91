// encode.cu -- the compression hot path on sm_100a: one warp per chunk.
//
// Steps (§3.2(2) "The GPU allocates multiple
// threads for each chunk. Each stage performs its own LZ compression algorithm
// with its own history buffer and look-ahead buffer."):
//   a2  stage the chunk (= its whole history window, R2) into shared memory with
//       a 1-D bulk TMA copy (cp.async.bulk + mbarrier).
//   a3  index: exact candidates of p are the earlier positions with the same
//       first k = min(m,4) bytes (a match of length >= m >= k starts with them).
//       The warp counting-sorts positions by a hash of that key into buckets
//       kept in ascending position order (stable scatter, MATCH.ANY ranks); bit
//       15 of an entry marks the first entry of its bucket.  A per-position bit
//       says whether a same-key position exists inside the window, and a
//       "byte changes here" bitmap gives run lengths in O(1) for the run
//       shortcut below.
//   a3  longest match at a token start p: the 32 lanes take the 32 nearest
//       candidates (slots below p's own), compute the capped common-prefix
//       length with 16-byte compares (or, when both sides start inside runs of
//       the same byte, straight from the two run lengths), pack
//       (len << 16 | 0xFFFF - (d-1)) and reduce with REDUX.MAX = "longest, then
//       nearest" (R6, R7).  A farther candidate must also match the byte at the
//       best length so far to be strictly longer, so most cost one compare.
//       Stop at the cap (exact: nothing beats it) or when bucket/window end.
//   a4  greedy walk (R8): literal runs advance up to 32 positions per step via
//       the candidate bitmap; the walk only records token starts, match bits,
//       (d-1) and (l-m) in place and keeps the running stream size, so a chunk
//       whose stream reaches n bytes is stored raw (R9) without encoding.
//   a5  encode (R1) in parallel over positions: token index and match count by
//       ballot/popc prefix sums give every token's output byte position; the
//       stream is assembled in shared memory and written with 16-byte stores.
// The serial result is reproduced exactly: the best match at p depends only on
// (chunk bytes, p, W, m, M), not on the parse.
#include "lzr_internal.cuh"

namespace lzr {

namespace {

constexpr int kMaxWarps = 16;
constexpr uint16_t kFirst = 0x8000;  // first entry of its bucket
constexpr uint16_t kPos = 0x7FFF;
constexpr uint32_t kMaxRuns = 32;  // runs of one byte value of length >= k, per chunk

__device__ __forceinline__ uint32_t khash(uint32_t key, uint32_t hbits) {
  return (key * 0x9E3779B1u) >> (32 - hbits);
}

// Common-prefix length of data[a..] and data[b..], capped at maxlen; 16 bytes
// per step (5 aligned words per side + funnel shifts).  Overlap (a > b) is
// allowed: original bytes are compared (= byte-serial copy semantics, R5).
__device__ __forceinline__ uint32_t lcp16(const uint8_t* d, uint32_t a, uint32_t b,
                                          uint32_t maxlen) {
  const uint32_t* w = reinterpret_cast<const uint32_t*>(d);
  const uint32_t sa = (a & 3u) << 3, sb = (b & 3u) << 3;
  uint32_t ia = a >> 2, ib = b >> 2;
  uint32_t a0 = w[ia], b0 = w[ib];
  uint32_t l = 0;
  while (l < maxlen) {
    const uint32_t a1 = w[ia + 1], a2 = w[ia + 2], a3 = w[ia + 3], a4 = w[ia + 4];
    const uint32_t b1 = w[ib + 1], b2 = w[ib + 2], b3 = w[ib + 3], b4 = w[ib + 4];
    const uint32_t x0 = __funnelshift_r(a0, a1, sa) ^ __funnelshift_r(b0, b1, sb);
    const uint32_t x1 = __funnelshift_r(a1, a2, sa) ^ __funnelshift_r(b1, b2, sb);
    const uint32_t x2 = __funnelshift_r(a2, a3, sa) ^ __funnelshift_r(b2, b3, sb);
    const uint32_t x3 = __funnelshift_r(a3, a4, sa) ^ __funnelshift_r(b3, b4, sb);
    if (x0 | x1 | x2 | x3) {
      uint32_t k, x;
      if (x0) { k = 0; x = x0; }
      else if (x1) { k = 4; x = x1; }
      else if (x2) { k = 8; x = x2; }
      else { k = 12; x = x3; }
      l += k + ((uint32_t)(__ffs(x) - 1) >> 3);
      return l < maxlen ? l : maxlen;
    }
    l += 16;
    ia += 4;
    ib += 4;
    a0 = a4;
    b0 = b4;
  }
  return maxlen;
}

// lcp16 for the common call (p-side start fixed for all lanes): the first 16
// p-side bytes are preloaded once per search (pw).
__device__ __forceinline__ uint32_t lcp16_pre(const uint8_t* d, const uint32_t (&pw)[4], uint32_t p,
                                              uint32_t q, uint32_t maxlen) {
  const uint32_t* w = reinterpret_cast<const uint32_t*>(d);
  const uint32_t sb = (q & 3u) << 3, ib = q >> 2;
  const uint32_t b0 = w[ib], b1 = w[ib + 1], b2 = w[ib + 2], b3 = w[ib + 3], b4 = w[ib + 4];
  const uint32_t x0 = pw[0] ^ __funnelshift_r(b0, b1, sb);
  const uint32_t x1 = pw[1] ^ __funnelshift_r(b1, b2, sb);
  const uint32_t x2 = pw[2] ^ __funnelshift_r(b2, b3, sb);
  const uint32_t x3 = pw[3] ^ __funnelshift_r(b3, b4, sb);
  const uint64_t lo = ((uint64_t)x1 << 32) | x0, hi = ((uint64_t)x3 << 32) | x2;
  uint32_t l;
  if (lo) l = (uint32_t)(__ffsll((long long)lo) - 1) >> 3;
  else if (hi) l = 8 + ((uint32_t)(__ffsll((long long)hi) - 1) >> 3);
  else l = maxlen > 16 ? 16 + lcp16(d, p + 16, q + 16, maxlen - 16) : 16;
  return l < maxlen ? l : maxlen;
}

// min(run length of the byte at p, lim): distance to the next set bit of the
// change bitmap cb (bit i = x[i] != x[i-1]; set for i >= n).
__device__ __forceinline__ uint32_t run_len(const uint32_t* cb, uint32_t p, uint32_t lim) {
  uint32_t i = p + 1;
  uint32_t wi = i >> 5;
  uint32_t bits = cb[wi] >> (i & 31u);
  uint32_t base = i;
  while (bits == 0) {
    ++wi;
    base = wi << 5;
    if (base - p >= lim) return lim;
    bits = cb[wi];
  }
  const uint32_t r = base + (uint32_t)(__ffs(bits) - 1) - p;
  return r < lim ? r : lim;
}

struct Smem {
  uint8_t* data;
  uint16_t* sorted;  // entries: position | kFirst; later: the output stream staging
  uint16_t* slot;    // histogram/cursors during the sort; slot of each position;
                     // after the walk: (d-1) at a match start, (l-m) right after it
  uint32_t* cand;    // 1: a same-key position exists inside the window
  uint32_t* cb;      // 1: byte differs from the previous one (run boundaries)
  uint32_t* tg;      // match toggles: bit s+1 and bit s+l for a match (s, l);
                     // prefix parity = "inside a match", so token starts and
                     // match starts follow without recording literals
  uint8_t* flags;    // flag byte of each group of 8 tokens
  uint32_t* runs;    // (end << 16) | start of every run of >= k equal bytes (first kMaxRuns)
};

// ---- a3: index ----------------------------------------------------------------
// Returns true when the chunk is certainly stored raw (R9) and the index was not
// built.  Sound bound: a match of length l at p makes positions p..p+l-k
// (k = key bytes) positions with a same-key earlier occurrence, disjoint across
// matches; with X = sum(l - 3) and T tokens, S = n - X + ceil(T/8) and
// T >= n - 3X (m >= 4) or n - 2(X + M) (m = 3), so S >= n whenever
// 11 * #{positions whose key hash was seen before} <= n.
__device__ __forceinline__ bool build_index(const Smem& S, uint32_t n, uint32_t P, const EncArgs& a,
                                            uint32_t lane, uint32_t& nruns) {
  const uint8_t* data = S.data;
  const uint32_t hb = a.L.hbits;
  const uint32_t B = 1u << hb;
  const uint32_t nw = a.L.bm_words;
  const uint32_t fb = a.L.fbits;
  uint32_t* hist = reinterpret_cast<uint32_t*>(S.slot);  // B u16 counters, two per word
  uint32_t* seen = reinterpret_cast<uint32_t*>(S.sorted);  // 2^fb-bit filter (index unused yet)
  for (uint32_t i = lane; i < B / 2; i += 32) hist[i] = 0;
  for (uint32_t i = lane; i < (1u << (fb - 5)); i += 32) seen[i] = 0;
  __syncwarp();
  // histogram of bucket sizes + "key hash seen before" count + run starts
  uint32_t U = 0, nr = 0;
  const uint32_t lt = lanemask_lt();
  for (uint32_t p0 = 0; p0 < P; p0 += 32) {
    const uint32_t p = p0 + lane;
    bool dup = false, rs = false;
    if (p < P) {
      const uint32_t key = ld32u(data, p) & a.kmask;
      const uint32_t h = khash(key, hb);
      atomicAdd(&hist[h >> 1], 1u << ((h & 1u) << 4));
      const uint32_t g = (key * 0x85EBCA6Bu) >> (32 - fb);
      dup = atomicOr(&seen[g >> 5], 1u << (g & 31u)) & (1u << (g & 31u));
      rs = ((key ^ (key >> 8)) & (a.kmask >> 8)) == 0 && (p == 0 || data[p - 1] != data[p]);
    }
    U += __popc(__ballot_sync(kFull, dup));
    const uint32_t rb = __ballot_sync(kFull, rs);
    const uint32_t idx = nr + __popc(rb & lt);
    if (rs && idx < kMaxRuns) S.runs[idx] = p;
    nr += __popc(rb);
  }
  nruns = nr;
  if (11u * U <= n) return true;
  for (uint32_t i = lane; i < nw; i += 32) {
    S.tg[i] = 0;
    S.cand[i] = 0;
  }
  for (uint32_t i = lane; i < a.C / 8; i += 32) S.flags[i] = 0;
  for (uint32_t w = 0; w < nw; ++w) {  // change bitmap
    const uint32_t i = (w << 5) + lane;
    const bool ch = (i == 0) || (i >= n) || (data[i] != data[i - 1]);
    const uint32_t b = __ballot_sync(kFull, ch);
    if (lane == 0) S.cb[w] = b;
  }
  __syncwarp();
  for (uint32_t j = lane; j < min(nruns, kMaxRuns); j += 32) {  // run ends
    const uint32_t st = S.runs[j];
    S.runs[j] = ((st + run_len(S.cb, st, n - st)) << 16) | st;
  }
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
  // stable scatter, 4 blocks of 32 positions per round so that the MATCH.ANY
  // latencies overlap; cursor updates stay in position order
  uint16_t* cur = S.slot;
  
  for (uint32_t p0 = 0; p0 < P; p0 += 128) {
    uint32_t h[4], peers[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t p = p0 + 32 * u + lane;
      h[u] = p < P ? khash(ld32u(data, p) & a.kmask, hb) : 0xFFFFFFFFu;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) peers[u] = __match_any_sync(kFull, h[u]);
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t p = p0 + 32 * u + lane;
      const bool act = p < P;
      const uint32_t basev = act ? cur[h[u]] : 0;
      if (act) S.sorted[basev + __popc(peers[u] & lt)] = (uint16_t)p;
      __syncwarp();
      if (act && lane == 31u - __clz(peers[u])) cur[h[u]] = (uint16_t)(basev + __popc(peers[u]));
      __syncwarp();
    }
  }
  // mark the first entry of every non-empty bucket (cur[h] = end of bucket h now)
  for (uint32_t hh = lane; hh < B; hh += 32) {
    const uint32_t st = hh ? cur[hh - 1] : 0u;
    if (cur[hh] > st) S.sorted[st] |= kFirst;
  }
  __syncwarp();
  // slot of each position (cursors are dead now) and the candidate bitmap: the
  // nearest same-key earlier position is the nearest same-key entry below in
  // the bucket; it decides whether a candidate lies inside the window
  for (uint32_t sl = lane; sl < P; sl += 32) {
    const uint32_t e = S.sorted[sl];
    const uint32_t q = e & kPos;
    S.slot[q] = (uint16_t)sl;
    if (!(e & kFirst)) {
      const uint32_t kq = ld32u(data, q) & a.kmask;
      bool has = false;
      for (uint32_t s2 = sl - 1;; --s2) {
        const uint32_t e2 = S.sorted[s2];
        const uint32_t q2 = e2 & kPos;
        if ((ld32u(data, q2) & a.kmask) == kq) {
          has = q - q2 <= a.W;
          break;
        }
        if (e2 & kFirst) break;
      }
      if (has) atomicOr(&S.cand[q >> 5], 1u << (q & 31u));
    }
  }
  __syncwarp();
  return false;
}

// ---- a3: longest, then nearest, capped match at p ------------------------------
// Run-aware exact search for a position p whose key is one repeated byte b and
// whose whole prefix lies in the window.  Every same-key candidate lies in a run
// of b; with r = min(run length at p, cap), a candidate q with run length
// RL(q) != r matches min(r, RL(q)) bytes and one with RL(q) == r matches
// r + (common prefix after both runs).  So in an earlier run [s, e) of b the
// best candidate, and the nearest among equals, is q = e - r when e - s >= r,
// else q = s with length e - s; inside p's own run it is d = 1 with length r.
// One lane per earlier run therefore decides the whole chunk history.
__device__ __forceinline__ uint32_t best_match_runs(const Smem& S, uint32_t p, uint32_t n,
                                                    uint32_t cap, uint32_t kp, uint32_t nruns,
                                                    const EncArgs& a, uint32_t lane) {
  const uint8_t* data = S.data;
  const uint32_t b = kp & 0xFFu;
  const uint32_t r = run_len(S.cb, p, cap);  // >= k
  uint32_t best = 0;
  if (p >= 1 && data[p - 1] == b && r >= a.m) best = (r << 16) | 0xFFFFu;  // d = 1
  for (uint32_t j0 = 0; j0 < nruns; j0 += 32) {
    const uint32_t j = j0 + lane;
    uint32_t pk = 0;
    if (j < nruns) {
      const uint32_t rr = S.runs[j];
      const uint32_t st = rr & 0xFFFFu, e = rr >> 16;
      if (data[st] == b) {
        const bool reach = e - st >= r;
        const uint32_t q = reach ? e - r : st;
        if (q < p) {
          const uint32_t l = !reach ? e - st : (r < cap ? r + lcp16(data, p + r, e, cap - r) : cap);
          if (l >= a.m) pk = (l << 16) | (0xFFFFu - (p - q - 1));
        }
      }
    }
    best = max(best, __reduce_max_sync(kFull, pk));
  }
  return best;
}

// Returns (len << 16) | (0xFFFF - (d-1)), or 0 when no candidate reaches m.
__device__ __forceinline__ uint32_t best_match(const Smem& S, uint32_t p, uint32_t n,
                                               uint32_t nruns, const EncArgs& a, uint32_t lane) {
  const uint8_t* data = S.data;
  const uint32_t cap = min(a.M, n - p);  // p < n - m + 1  =>  cap >= m >= k
  const uint32_t kp = ld32u(data, p) & a.kmask;
  const bool prun = ((kp ^ (kp >> 8)) & (a.kmask >> 8)) == 0;  // key = one repeated byte
  const bool all_in_window = p <= a.W;
  if (prun && all_in_window && nruns <= kMaxRuns)
    return best_match_runs(S, p, n, cap, kp, nruns, a, lane);
  // run shortcut for the generic path (window smaller than the prefix / many runs)
  const uint32_t rp = prun ? run_len(S.cb, p, cap) : 0u;
  uint32_t pw[4];
  {
    const uint32_t* w = reinterpret_cast<const uint32_t*>(data);
    const uint32_t sa = (p & 3u) << 3, ia = p >> 2;
    const uint32_t a0 = w[ia], a1 = w[ia + 1], a2 = w[ia + 2], a3 = w[ia + 3], a4 = w[ia + 4];
    pw[0] = __funnelshift_r(a0, a1, sa);
    pw[1] = __funnelshift_r(a1, a2, sa);
    pw[2] = __funnelshift_r(a2, a3, sa);
    pw[3] = __funnelshift_r(a3, a4, sa);
  }
  uint32_t best = 0, blen = 0;
  int sb = (int)S.slot[p] - 1;  // the walk only asks at positions with a candidate
  for (;; sb -= 32) {
    const int s = sb - (int)lane;
    uint32_t e = kFirst, q = 0;
    bool ok = s >= 0;
    if (ok) {
      e = S.sorted[s];
      q = e & kPos;
      ok = all_in_window || p - q <= a.W;
    }
    // lanes up to and including the bucket's first entry, and inside the window
    const uint32_t m_first = __ballot_sync(kFull, ok && (e & kFirst));
    const uint32_t m_stop = __ballot_sync(kFull, !ok);
    uint32_t lim = 32;
    if (m_first) lim = (uint32_t)__ffs(m_first);
    if (m_stop) lim = min(lim, (uint32_t)(__ffs(m_stop) - 1));
    uint32_t pk = 0;
    if (lane < lim && (blen == 0 || data[q + blen] == data[p + blen])) {
      uint32_t l;
      if (rp) {
        if ((ld32u(data, q) & a.kmask) != kp) {
          l = 0;  // hash collision
        } else {
          const uint32_t rq = run_len(S.cb, q, cap);
          l = rq != rp ? min(rp, rq) : (rp < cap ? rp + lcp16(data, p + rp, q + rp, cap - rp) : cap);
        }
      } else {
        l = lcp16_pre(data, pw, p, q, cap);
      }
      if (l >= a.m) pk = (l << 16) | (0xFFFFu - (p - q - 1));
    }
    best = max(best, __reduce_max_sync(kFull, pk));
    blen = best >> 16;
    if (blen >= cap || lim < 32) break;
  }
  return best;
}

// ---- a5: parallel encode of the recorded parse into the staging buffer --------
// inside(t) = parity of match toggles at positions <= t; token starts are the
// positions not inside a match, match starts s have inside(s) = 0, inside(s+1) = 1.
__device__ __forceinline__ uint32_t prefix_parity(uint32_t x) {
  x ^= x << 1;
  x ^= x << 2;
  x ^= x << 4;
  x ^= x << 8;
  x ^= x << 16;
  return x;
}

__device__ __forceinline__ void encode_tokens(const Smem& S, uint32_t n, uint8_t* ob, uint32_t lane) {
  const uint32_t lt = lanemask_lt();
  uint32_t carryT = 0, carryM = 0, par = 0;
  const uint32_t nwords = (n + 31) >> 5;
  uint32_t tg_next = S.tg[0];
  for (uint32_t w = 0; w < nwords; ++w) {
    const uint32_t tgw = tg_next;
    tg_next = S.tg[w + 1];
    const uint32_t inside = prefix_parity(tgw) ^ (0u - par);
    par = inside >> 31;
    const uint32_t next0 = par ^ (tg_next & 1u);
    const uint32_t valid = (n - (w << 5)) >= 32 ? 0xFFFFFFFFu : ((1u << (n - (w << 5))) - 1u);
    const uint32_t tw = ~inside & valid;
    const uint32_t mw = ~inside & ((inside >> 1) | (next0 << 31)) & valid;
    const uint32_t p = (w << 5) + lane;
    if ((tw >> lane) & 1u) {
      const uint32_t j = carryT + __popc(tw & lt);
      const uint32_t mbef = carryM + __popc(mw & lt);
      const uint32_t pos = j + 2 * mbef + (j >> 3) + 1;
      if ((j & 7u) == 0) ob[pos - 1] = S.flags[j >> 3];
      if ((mw >> lane) & 1u) {
        const uint32_t dm1 = S.slot[p], lm = S.slot[p + 1];
        ob[pos] = (uint8_t)(dm1 & 0xFF);
        ob[pos + 1] = (uint8_t)(dm1 >> 8);
        ob[pos + 2] = (uint8_t)lm;
      } else {
        ob[pos] = S.data[p];
      }
    }
    carryT += __popc(tw);
    carryM += __popc(mw);
  }
}

__global__ void __launch_bounds__(32 * kMaxWarps, 1) lzr_encode_kernel(const EncArgs a) {
  extern __shared__ __align__(128) uint8_t smem[];
  const uint32_t lane = threadIdx.x & 31u;
  const uint32_t warp = threadIdx.x >> 5;
  uint8_t* base = smem + (size_t)warp * a.L.per_warp;
  Smem S;
  S.data = base;
  S.sorted = reinterpret_cast<uint16_t*>(base + a.L.off_sorted);
  S.slot = reinterpret_cast<uint16_t*>(base + a.L.off_slot);
  uint32_t* bms = reinterpret_cast<uint32_t*>(base + a.L.off_bm);
  const uint32_t nw = a.L.bm_words;
  S.cand = bms;
  S.cb = bms + nw;
  S.tg = bms + 2 * nw;
  S.flags = reinterpret_cast<uint8_t*>(bms + 4 * nw);
  S.runs = reinterpret_cast<uint32_t*>(S.flags + align_up(a.C / 8, 4));
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
      tma_bulk_g2s(S.data, src, n16, bar);
    }
    for (uint32_t i = n16 + lane; i < n; i += 32) S.data[i] = src[i];
    for (uint32_t i = n + lane; i < align_up(n, 16) + 32; i += 32) S.data[i] = 0;
    if (n16) {
      mbar_wait_parity(bar, phase);
      phase ^= 1u;
    }
    __syncwarp();

    const uint32_t P = n >= a.m ? n - a.m + 1 : 0;  // positions that can start a match
    uint32_t nruns = 0;
    bool raw = build_index(S, n, P, a, lane, nruns);

    // ---- a3/a4: greedy walk.  Only matches are recorded (toggles, (d-1), (l-m));
    // literal runs just advance p and the token count T; the flag byte of the
    // current group of 8 tokens accumulates in a register.
    uint32_t T = 0, Mt = 0;
    uint32_t p = 0;
    uint32_t gcur = 0, acc_f = 0;
    while (!raw && p < n) {
      uint32_t bits = 0;
      if (p < P) bits = __funnelshift_r(S.cand[p >> 5], S.cand[(p >> 5) + 1], p & 31u);
      if (bits == 0) {  // 32 (or the rest) literals
        const uint32_t L = min(32u, n - p);
        T += L;
        p += L;
      } else {
        const uint32_t f = (uint32_t)(__ffs(bits) - 1);  // literals before the candidate
        T += f;
        p += f;
        const uint32_t r = best_match(S, p, n, nruns, a, lane);
        const uint32_t l = r >> 16;
        if (l >= a.m) {
          if (lane == 0) {
            atomicOr(&S.tg[(p + 1) >> 5], 1u << ((p + 1) & 31u));
            atomicOr(&S.tg[(p + l) >> 5], 1u << ((p + l) & 31u));
            S.slot[p] = (uint16_t)(0xFFFFu - (r & 0xFFFFu));  // d - 1
            S.slot[p + 1] = (uint16_t)(l - a.m);
          }
          if ((T >> 3) != gcur) {
            if (lane == 0 && acc_f) S.flags[gcur] = (uint8_t)acc_f;
            gcur = T >> 3;
            acc_f = 0;
          }
          acc_f |= 1u << (T & 7u);
          Mt += 1;
          p += l;
        } else {
          p += 1;
        }
        T += 1;
      }
      if (T + 2 * Mt + ((T + 7) >> 3) >= n) raw = true;  // not shorter than the chunk (R9)
    }
    if (!raw && lane == 0 && acc_f) S.flags[gcur] = (uint8_t)acc_f;
    __syncwarp();
    uint32_t Sz = n;
    if (!raw) {
      Sz = T + 2 * Mt + ((T + 7) >> 3);
      uint8_t* ob = reinterpret_cast<uint8_t*>(S.sorted);  // the index is dead now
      encode_tokens(S, n, ob, lane);
      __syncwarp();
      uint8_t* out = a.slots + lo;
      const uint32_t n16o = align_up(Sz, 16);
      for (uint32_t i = lane * 16; i < n16o; i += 32 * 16)
        *reinterpret_cast<uint4*>(out + i) = *reinterpret_cast<const uint4*>(ob + i);
    }
    if (lane == 0) a.sizes[c] = Sz;
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
