// encode.cu -- the compression hot path on sm_100a: K warps per chunk.
//
// Steps (§3.2(2) "The GPU allocates multiple
// threads for each chunk. Each stage performs its own LZ compression algorithm
// with its own history buffer and look-ahead buffer. Adjacent threads inspect
// overlapping regions by the size of the history buffer."):
//   a2  stage the chunk (= its whole history window, R2) into shared memory with
//       a 1-D bulk TMA copy (cp.async.bulk + mbarrier).
//   a3  index (the group's K warps share the passes): exact candidates of p are
//       the earlier positions with the same first k = min(m,4) bytes (a match
//       of length >= m >= k starts with them).  Positions are counting-sorted
//       by a hash of that key into buckets kept in ascending position order
//       (stable scatter, MATCH.ANY ranks); bit 15 of an entry marks the first
//       entry of its bucket.  A candidate bitmap says whether a same-key
//       position exists inside the window; a byte-change bitmap and a run list
//       serve the run-aware search.  A sound pre-filter proves most
//       incompressible chunks raw before any of this.
//   a3  longest match at a token start p (one warp): the 32 lanes take the 32
//       nearest candidates, compute capped common-prefix lengths with 16-byte
//       compares, pack (len << 16 | 0xFFFF - (d-1)) and reduce with REDUX.MAX =
//       "longest, then nearest" (R6, R7); positions whose key is one repeated
//       byte use the exact run-aware search instead.
//   a4  greedy walk (R8), split into K speculative segments: warp k parses from
//       k*n/K.  Greedy parses are deterministic, so two parses that share one
//       token start coincide from there on; warp k stops at the first of its
//       token starts that warp k+1 has also recorded, and the exact serial parse
//       is the chain warp 0 -> warp 1 -> ... through those meeting points (the
//       paper's overlapping per-thread regions, made exact).  The parse is kept
//       as a token-start bitmap plus (d-1) at each match start.
//   a5  encode (R1) in parallel over positions: a token is a match iff the next
//       token starts more than one byte later; token index and match count by
//       popc prefix sums give every token's byte position; the stream is staged
//       in shared memory and written with 16-byte stores; raw fallback (R9).
// The serial result is reproduced exactly: the best match at p depends only on
// (chunk bytes, p, W, m, M), not on the parse.
#include <mutex>

#include "lzr_internal.cuh"

namespace lzr {

namespace {

constexpr uint16_t kFirst = 0x8000;  // first entry of its bucket
constexpr uint16_t kPos = 0x7FFF;

// ctrl word indices (per group): chunk, U, nruns, then prog[K], sync[K] during
// the walk, reused as T[K], M[K] (token / match totals) after the chain phase
constexpr int kCtrlChunk = 0, kCtrlU = 1, kCtrlRuns = 2, kCtrlIdx = 3, kCtrlProg = 4;

// Bucket of a key.  With >= 1024 buckets, keys that are one repeated byte get
// private buckets 0..255 (their buckets can hold thousands of positions, e.g.
// zero runs, and a colliding key would scan them all); other keys hash into
// the remaining B - 256.
__device__ __forceinline__ uint32_t khash(uint32_t key, uint32_t hbits, uint32_t kmask) {
  const uint32_t h = (key * 0x9E3779B1u) >> (32 - hbits);
  if (hbits < 10) return h;
  if (((key ^ (key >> 8)) & (kmask >> 8)) == 0) return key & 0xFFu;
  return 256u + ((h * ((1u << hbits) - 256u)) >> hbits);
}

__device__ __forceinline__ void group_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

#ifdef LZR_PHASE_TIMING
// debug build only: per phase and warp-in-group, cycles working / waiting at
// the group barrier that closes the phase
__device__ unsigned long long g_phase[16][4][2];
#define GSYNC(ph)                                                            \
  do {                                                                       \
    const long long t_arr = clock64();                                       \
    group_sync(bar_id, nthr);                                                \
    const long long t_lv = clock64();                                        \
    if (lane == 0) {                                                         \
      atomicAdd(&g_phase[ph][k & 3][0], (unsigned long long)(t_arr - t_ph)); \
      atomicAdd(&g_phase[ph][k & 3][1], (unsigned long long)(t_lv - t_arr)); \
    }                                                                        \
    t_ph = t_lv;                                                             \
  } while (0)
#else
#define GSYNC(ph) group_sync(bar_id, nthr)
#endif

// predicated shared-memory OR without a returned value (no branch, no wait)
__device__ __forceinline__ void red_or_if(bool pred, uint32_t* addr, uint32_t v) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %0, 0;\n\t@q red.shared.or.b32 [%1], %2;\n\t}" ::"r"(
          (uint32_t)pred),
      "r"(smem_u32(addr)), "r"(v)
      : "memory");
}
// token-start bits of a walk segment: shared memory, or (big chunks) the
// group's global scratch
template <bool BIG>
__device__ __forceinline__ void tb_or_if(bool pred, uint32_t* addr, uint32_t v) {
  if (BIG) {
    if (pred) atomicOr(addr, v);
  } else {
    red_or_if(pred, addr, v);
  }
}
// predicated 16-bit global store
__device__ __forceinline__ void st_u16_if(bool pred, uint16_t* addr, uint32_t v) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %0, 0;\n\t@q st.global.u16 [%1], %2;\n\t}" ::"r"(
          (uint32_t)pred),
      "l"(addr), "h"((uint16_t)v)
      : "memory");
}

__device__ __forceinline__ void fence_acq_rel_cta() {
  asm volatile("fence.acq_rel.cta;" ::: "memory");
}

__device__ __forceinline__ uint32_t ld_volatile(const uint32_t* p) {
  return *reinterpret_cast<const volatile uint32_t*>(p);
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
    const uint64_t lo = ((uint64_t)x1 << 32) | x0, hi = ((uint64_t)x3 << 32) | x2;
    if (lo | hi) {
      l += lo ? ((uint32_t)(__ffsll((long long)lo) - 1) >> 3)
              : 8 + ((uint32_t)(__ffsll((long long)hi) - 1) >> 3);
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

// Shared memory of one group (one chunk in flight).
struct Smem {
  uint8_t* data;
  uint16_t* sorted;  // entries: position | kFirst; after the walk: output staging
  uint16_t* slot;    // histogram/cursors during the sort; slot of each position
  uint32_t* cand;    // 1: a same-key position exists inside the window;
                     // after the walk: the final token-start bitmap (+ bit n)
  uint32_t* cb;      // 1: byte differs from the previous one (run boundaries);
                     // after the walk: match bit per token index (flag bytes)
  uint32_t* tb;      // K token-start bitmaps, one per walk segment
  uint32_t* runs;    // ((end - 1) << 16) | start of every run of >= k equal bytes
  uint32_t* ctrl;    // chunk, U, nruns, prog[K], sync[K], T[K], M[K]
  uint64_t* bar;
};

// ---- a3: longest, then nearest, capped match at p ------------------------------
// Run-aware exact search for a position p whose key is one repeated byte b and
// whose whole prefix lies in the window.  Every same-key candidate lies in a run
// of b; with r = min(run length at p, cap), a candidate q with run length
// RL(q) != r matches min(r, RL(q)) bytes and one with RL(q) == r matches
// r + (common prefix after both runs).  So in an earlier run [s, e) of b the
// best candidate, and the nearest among equals, is q = e - r when e - s >= r,
// else q = s with length e - s; inside p's own run it is d = 1 with length r.
// One lane per earlier run therefore decides the whole chunk history.
__device__ __forceinline__ uint32_t best_match_runs(const Smem& S, uint32_t p, uint32_t cap,
                                                    uint32_t kp, uint32_t nruns, const EncArgs& a,
                                                    uint32_t lane) {
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
      const uint32_t st = rr & 0xFFFFu, e = (rr >> 16) + 1u;  // run [st, e)
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
// floor > 0 (lazy parse only asks whether some match is longer than floor):
// the generic path then evaluates only candidates that also match the byte at
// offset floor; the result is exact whenever it exceeds floor (every candidate
// reaching the maximum passes that test), otherwise it is some value <= floor.
// prevb <= 0xFF (lazy parse, p = q0 + 1 after a match of length floor < cap at
// q0, prevb = x[q0]): a candidate r preceded by prevb (x[r-1] == x[q0]) is
// skipped -- r - 1 then has q0's key at the same distance, so it is a
// candidate of q0, whose best length floor is below q0's cap; hence
// LCP(q0, r-1) <= floor and LCP(p, r) = LCP(q0, r-1) - 1 < floor.
template <bool BIG>
__device__ __forceinline__ uint32_t best_match(const Smem& S, uint32_t p, uint32_t n,
                                               uint32_t nruns, const EncArgs& a, uint32_t lane,
                                               uint32_t floor = 0, uint32_t prevb = 0x100u) {
  const uint8_t* data = S.data;
  const uint32_t cap = min(a.M, n - p);  // p < n - m + 1  =>  cap >= m >= k
  const uint32_t kp = ld32u(data, p) & a.kmask;
  const bool prun = ((kp ^ (kp >> 8)) & (a.kmask >> 8)) == 0;  // key = one repeated byte
  const bool all_in_window = p <= a.W;
  if (prun && all_in_window && nruns <= a.L.max_runs)
    return best_match_runs(S, p, cap, kp, nruns, a, lane);
  // (generic path: window smaller than the prefix, many runs, or a plain key).
  // One candidate per lane, nearest first, 32 per round; p's first 16 bytes
  // are preloaded for the 16-byte compares.  (A separate path for lists of
  // <= 8 candidates -- 4-8 lanes per candidate -- and 64 candidates per round
  // both measured slower: mix 52.3 vs 51.0 / 51.5 GB/s.)
  uint32_t best = 0, blen = floor;
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
  // p's own index entry (the walk only asks at positions with a candidate, so
  // p is indexed); the candidates are the entries of its bucket below it
  int sb0, bstart = 0;
  if (BIG) {
    // big chunks: no slot array -- find p inside its bucket [bs, be) (entries
    // ascending) by a 32-ary search, lane i probing lo + i * step
    const uint16_t* ends = S.slot + (a.L.nsplit - 1) * (1u << a.L.hbits);  // the last split's cursors
    const uint32_t h = khash(kp, a.L.hbits, a.kmask);
    const uint32_t bs = h ? ends[h - 1] : 0u;
    uint32_t lo = bs, hi = ends[h];  // p in [lo, hi), sorted[lo] <= p
#ifdef LZR_WATCHDOG
    uint32_t spins = 0;
#endif
    while (hi - lo > 32u) {
      LZR_SPIN_GUARD(spins, "bucket search")
      const uint32_t step = (hi - lo + 31u) >> 5;
      const uint32_t idx = lo + lane * step;
      const uint32_t bal = __ballot_sync(kFull, idx < hi && S.sorted[idx] <= p);
      lo += (31u - __clz(bal)) * step;
      hi = min(hi, lo + step);
    }
    const uint32_t bal = __ballot_sync(kFull, lo + lane < hi && S.sorted[lo + lane] <= p);
    sb0 = (int)(lo + 31u - __clz(bal));
    bstart = (int)bs;
  } else {
    sb0 = (int)S.slot[p];
  }
  for (int sb = sb0 - 1;; sb -= 32) {
    const int s = sb - (int)lane;
    uint32_t e = kFirst, q = 0;
    bool ok = s >= bstart;
    if (ok) {
      e = S.sorted[s];
      q = BIG ? e : e & kPos;
      ok = all_in_window || p - q <= a.W;
    }
    // lanes up to and including the bucket's first entry, and inside the window
    const uint32_t m_first = BIG ? 0u : __ballot_sync(kFull, ok && (e & kFirst));
    const uint32_t m_stop = __ballot_sync(kFull, !ok);
    uint32_t lim = 32;
    if (m_first) lim = (uint32_t)__ffs(m_first);
    if (m_stop) lim = min(lim, (uint32_t)(__ffs(m_stop) - 1));
    uint32_t pk = 0;
    if (lane < lim && (blen == 0 || data[q + blen] == data[p + blen]) &&
        (prevb > 0xFFu || q == 0 || data[q - 1] != prevb)) {
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
    blen = max(floor, best >> 16);
    if (blen >= cap || lim < 32) break;
  }
  return best;
}

// ---- a4: one speculative walk segment ----------------------------------------
// Warp k parses greedily from `start`.  Token starts go into its bitmap tbk
// (lane 0, atomics), (d-1) into d1[s] at each match start s (the group's global
// scratch; identical from every warp that records a token at s, since the best
// match at s does not depend on the parse).  prog[k]: every token start of warp k below prog[k] is
// recorded.  A warp with a successor stops at the first of its token starts x
// that the successor has recorded (x < prog[k+1]); sync[k] = x, or n if it ran
// to the end.
// LZ (one-step lazy parse, R21): a match at q is taken only if the best match
// at q + 1 is not strictly longer; otherwise q is a literal and the walk moves
// to q + 1, whose best match is then already known (cached).  The decision at
// q depends on q alone, so the meeting-point argument above is unchanged.
// zero-run block skipping in the scatter (4 KiB mix / text / zero-runs:
// 58.2 / 31.2 / 94.7 -> 59.2 / 30.9 / 105.3 GB/s)
#ifndef LZR_SKIPB
#define LZR_SKIPB 1
#endif
#ifndef LZR_PUB
#define LZR_PUB 64  // progress published every LZR_PUB bytes of parse
#endif
template <int K, bool LZ, bool BIG, bool TBG>
__device__ __forceinline__ void walk_segment(const Smem& S, uint16_t* d1, uint32_t k, uint32_t start,
                                             uint32_t nb, uint32_t n, uint32_t P, uint32_t nruns,
                                             const EncArgs& a, uint32_t lane) {
  const uint32_t tw = a.L.tb_words;
  uint32_t* tbk = S.tb + k * tw;
  const uint32_t* tbn = S.tb + (k + 1) * tw;  // successor's bitmap (k < K-1 only)
  uint32_t* prog = S.ctrl + kCtrlProg;
  uint32_t* sync = prog + K;
  uint32_t p = start, pub = start;
  uint32_t stop_at = n;
  uint32_t cq = 0xFFFFFFFFu, cr = 0;  // LZ: best match already computed at cq
#ifdef LZR_PHASE_TIMING
  long long t_bm = 0, n_bm = 0, n_it = 0;
#endif
#ifdef LZR_WATCHDOG
  uint32_t spins = 0;
#endif
  while (p < n) {
    LZR_SPIN_GUARD(spins, "walk")
#ifdef LZR_PHASE_TIMING
    ++n_it;
#endif
    // one iteration = the literal stretch before the next candidate position
    // q = p + L (from the candidate bitmap, up to 32 positions) and, if q was
    // found, the token at q
    uint32_t bits = 0;
    if (p < P) bits = __funnelshift_r(S.cand[p >> 5], S.cand[(p >> 5) + 1], p & 31u);
    const uint32_t L = bits ? (uint32_t)(__ffs(bits) - 1) : min(32u, n - p);
    const uint32_t q = p + L;
    uint32_t tok_len = 0, r = 0, cnt = L;  // cnt: token starts recorded, [p, p + cnt)
    if (bits) {
#ifdef LZR_PHASE_TIMING
      const long long tb0 = clock64();
#endif
      r = (LZ && q == cq) ? cr : best_match<BIG>(S, q, n, nruns, a, lane);
#ifdef LZR_PHASE_TIMING
      t_bm += clock64() - tb0;
      ++n_bm;
#endif
      uint32_t l = r >> 16;
      // LZ: a longer match at q + 1 is possible only if l is below its cap
      // min(M, n - q - 1) and q + 1 has a same-key candidate
      // A match longer than l at q + 1 covers the keys at s = q + l + 1 - k and
      // q + l + 2 - k (the keys that contain x[q + l], the byte that ended q's
      // match; k = key length), at its own distance: both then have a
      // candidate.  Either without one (and a candidate-tracked position,
      // < P) => no longer match at q + 1 => no search.
      const uint32_t s_lz = q + l + 1 - a.kbytes;
      const uint32_t two = __funnelshift_r(S.cand[s_lz >> 5], S.cand[(s_lz >> 5) + 1], s_lz & 31u) & 3u;
      if (LZ && l >= a.m && l < min(a.M, n - q - 1) && ((S.cand[(q + 1) >> 5] >> ((q + 1) & 31u)) & 1u) &&
          (s_lz + 1 >= P || two == 3u)) {
        cr = best_match<BIG>(S, q + 1, n, nruns, a, lane, l, S.data[q]);  // exact if > l
        cq = q + 1;
        if ((cr >> 16) > l) l = 0;  // deferred: x[q] is a literal
      }
      tok_len = l >= a.m ? l : 1u;
      cnt = L + 1;  // <= 32
    }
    // record token starts [p, p+cnt) and (d-1) at q (lane 0, predicated)
    {
      const uint32_t w = p >> 5, sh = p & 31u;
      const uint32_t mask = cnt >= 32 ? 0xFFFFFFFFu : ((1u << cnt) - 1u);
      tb_or_if<TBG>(lane == 0, &tbk[w], mask << sh);
      tb_or_if<TBG>(lane == 0 && sh + cnt > 32, &tbk[w + 1], sh ? mask >> (32 - sh) : 0u);
      st_u16_if(lane == 0 && tok_len > 1, d1 + q, 0xFFFFu - (r & 0xFFFFu));  // d - 1
    }
    // does this stretch meet the successor's parse?
    if (K > 1 && k + 1 < K && p + cnt > nb) {
      // one atomic read of the successor's progress, broadcast: per-lane reads
      // could see different values and split the warp (-> warp-sync deadlock)
      uint32_t pr = 0;
      if (lane == 0) {
        pr = atomicAdd(&prog[k + 1], 0u);
        fence_acq_rel_cta();  // the successor's bits below pr are visible after this
      }
      pr = __shfl_sync(kFull, pr, 0);
      const uint32_t lo = max(p, nb), hi = min(p + cnt, pr);
      if (lo < hi) {
        uint32_t x = hi;
        for (uint32_t w = lo >> 5; w <= (hi - 1) >> 5; ++w) {
          uint32_t b = 0;
          if (lane == 0) b = ld_volatile(&tbn[w]);
          b = __shfl_sync(kFull, b, 0);  // uniform across the warp (see above)
          const uint32_t wlo = w << 5;
          if (wlo < lo) b &= 0xFFFFFFFFu << (lo - wlo);
          if (hi - wlo < 32) b &= (1u << (hi - wlo)) - 1u;
          if (b) {
            x = wlo + (uint32_t)(__ffs(b) - 1);
            break;
          }
        }
        if (x < hi) {
          stop_at = x;
          if (lane == 0) {
            fence_acq_rel_cta();
            atomicExch(&prog[k], x + 1);
          }
          break;
        }
      }
    }
    p = bits ? q + tok_len : q;
    // publish progress (a later publish only delays meeting; warp 0's is never read)
    if (k > 0 && (p - pub >= LZR_PUB || p >= n)) {
      pub = p;
      if (lane == 0) {
        fence_acq_rel_cta();  // recorded token bits before the progress word
        atomicExch(&prog[k], p);
      }
    }
  }
  if (lane == 0) sync[k] = stop_at;
#ifdef LZR_PHASE_TIMING
  if (lane == 0) {
    atomicAdd(&g_phase[12][k & 3][0], (unsigned long long)t_bm);
    atomicAdd(&g_phase[12][k & 3][1], (unsigned long long)n_bm);
    atomicAdd(&g_phase[13][k & 3][1], (unsigned long long)n_it);
  }
#endif
}

__device__ __forceinline__ uint32_t walk_bound(uint32_t n, uint32_t k, uint32_t K) {
  if (k == 0) return 0;
  if (k >= K) return n;
#ifndef LZR_WALK_C
#define LZR_WALK_C 0.5f
#endif
  // work density 1 + c x over the chunk (later positions have more candidates)
  // => bound x solves x + c x^2 / 2 = (k/K)(1 + c/2)
  constexpr float c = LZR_WALK_C;
  const float f = (sqrtf(1.0f + 2.0f * c * (1.0f + 0.5f * c) * (float)k / (float)K) - 1.0f) / c;
  const uint32_t b = (uint32_t)(f * (float)n);
  return b < n ? b : n;
}

// (A/B on 1 x B200, 256 MiB, GB/s mix/text/zero-runs: fixed slope bounds
// 51.8/28.2/81.5; A:B = 2:1 52.3/28.5/81.0; 1:1 52.2; 1:2 52.2; 3:1 52.4; 4:1 52.2;
// 8:1 52.1.  LZR_WALK_CAND_A=0 restores walk_bound.)
#ifndef LZR_WALK_CAND_A
#define LZR_WALK_CAND_A 2u
#endif
#ifndef LZR_WALK_CAND_B
#define LZR_WALK_CAND_B 1u
#endif
// Segment bounds from the candidate bitmap (LZR_WALK_CAND_A > 0): a word of 32
// positions weighs A * (its candidate positions) + B (B ~ one literal-stretch
// iteration); bounds are word starts splitting the total weight into K equal
// parts.  Any bounds give the exact parse (meeting points), so this only moves
// work between the walk segments.
__device__ __forceinline__ uint32_t walk_bound_cand(const uint32_t* cand, uint32_t nwords,
                                                    uint32_t n, uint32_t kk, uint32_t K,
                                                    uint32_t tot, uint32_t lane) {
  if (kk == 0) return 0;
  if (kk >= K) return n;
  const uint32_t t = (uint32_t)(((unsigned long long)tot * kk) / K);
  uint32_t carry = 0;
  for (uint32_t w0 = 0; w0 < nwords; w0 += 32) {
    const uint32_t w = w0 + lane;
    const uint32_t v = w < nwords ? LZR_WALK_CAND_A * __popc(cand[w]) + LZR_WALK_CAND_B : 0u;
    uint32_t incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, incl, o);
      if ((int)lane >= o) incl += y;
    }
    // first word whose exclusive cumulative weight reaches t
    const uint32_t hit = __ballot_sync(kFull, w < nwords && carry + incl - v >= t);
    if (hit) return min(n, (w0 + (uint32_t)(__ffs(hit) - 1)) << 5);
    carry += __shfl_sync(kFull, incl, 31);
  }
  return n;
}

__device__ __forceinline__ uint32_t valid_mask(uint32_t n, uint32_t w) {
  const uint32_t base = w << 5;
  return n >= base + 32 ? 0xFFFFFFFFu : (n > base ? (1u << (n - base)) - 1u : 0u);
}

// threads per CTA at most (K = 1..3: 10 groups of 1 or 2 warps, 9 of 3)
// CTA shapes (A/B on 1 x B200, tools/ab.sh): K = 4 runs 3 CTAs of 3 groups per
// SM (9 groups = 36 warps at <= 56 registers; 1 CTA of 8 groups: mix 46.9 ->
// 50.1 GB/s, zero-runs 61.7 -> 71.7); K = 8 (C > 4 KiB) see LZR_K8_*.
#ifndef LZR_K4_THREADS
#define LZR_K4_THREADS 384
#endif
#ifndef LZR_K4_MINB
#define LZR_K4_MINB 3
#endif
#ifndef LZR_K8_THREADS
#define LZR_K8_THREADS 1024
#endif
#ifndef LZR_K8_MINB
#define LZR_K8_MINB 1
#endif
// G1: one group per CTA (K = 4 only; 9 CTAs of 4 warps per SM, same registers
// and occupancy).  Used for launches of few waves: a CTA then leaves the SM as
// soon as its one group runs out of chunks, so the tail of the launch (the last
// chunks, up to one chunk latency) overlaps the next launch on another stream
// instead of holding the SM (1 x B200, 16 MiB batches on 4 streams: 46.6 ->
// 50.8 GB/s; one 256 MiB launch: 51.9 -> 50.5, so large launches keep 3 x 3).
template <int K, bool G1 = false>
struct MaxThreads {
  static constexpr int value =
      G1 ? 32 * K
         : (K == 1 ? 320
                   : (K == 2 ? 640
                             : (K == 3 ? 864 : (K == 4 ? LZR_K4_THREADS : (K == 16 ? 512 : (K == 32 ? 1024 : LZR_K8_THREADS))))));
};
// K = 16 outside the big layout: 2 CTAs per SM (<= 64 registers) so that two
// 16 KiB chunks of 16 warps fit an SM; one 32 KiB chunk fills it anyway
#ifndef LZR_K16_MINB
#define LZR_K16_MINB 2
#endif
template <int K, bool G1 = false, bool BIG = false>
struct MinBlocks {
  static constexpr int value =
      G1 ? (K == 4 ? 9 : 1)
         : (K == 4 ? LZR_K4_MINB : (K == 8 ? LZR_K8_MINB : (K == 16 && !BIG ? LZR_K16_MINB : 1)));
};
#ifndef LZR_G1_MAX_WAVES
#define LZR_G1_MAX_WAVES 12u
#endif
constexpr uint32_t kG1MaxWaves = LZR_G1_MAX_WAVES;  // launches of fewer chunk waves than this use G1

// CF != 0: the kernel specialised for chunk size CF (the layout's offsets and
// sizes become compile-time constants); DEF: also for the configs' parameters
// W = C, m = 4, M = 259
template <int K, int NS, bool LZ, bool G1, bool BIG, uint32_t CF, bool DEF = false>
__global__ void __launch_bounds__(MaxThreads<K, G1>::value, MinBlocks<K, G1, BIG>::value)
    lzr_encode_kernel(const EncArgs a_in) {
  EncArgs a_fix = a_in;
  if (CF) {
    constexpr EncLayout LF = enc_layout(CF ? CF : 4096u, K, NS);
    a_fix.L = LF;
    a_fix.C = CF;
    if (DEF) {
      a_fix.W = CF;
      a_fix.m = 4;
      a_fix.M = 259;
      a_fix.kbytes = 4;
      a_fix.kmask = 0xFFFFFFFFu;
    }
  }
  const EncArgs& a = CF ? a_fix : a_in;
  extern __shared__ __align__(128) uint8_t smem[];
  const uint32_t lane = threadIdx.x & 31u;
  const uint32_t warp = threadIdx.x >> 5;
  const uint32_t g = warp / K, k = warp % K;  // group, warp within the group
  const uint32_t bar_id = 1 + g, nthr = 32 * K;
  uint8_t* base = smem + (size_t)g * a.L.per_group;
  const uint32_t nw = a.L.bm_words;
  Smem S;
  S.data = base;
  S.sorted = reinterpret_cast<uint16_t*>(base + a.L.off_sorted);
  S.slot = reinterpret_cast<uint16_t*>(base + a.L.off_slot);
  uint32_t* bms = reinterpret_cast<uint32_t*>(base + a.L.off_bm);
  S.cand = bms;
  S.cb = bms + nw;
  S.tb = bms + 2 * nw;  // (big chunks: in the global scratch, below)
  // token-start bitmaps of the walk segments in the global scratch: big chunks
  // and the 16- and 32-warp groups of chunks above 8 KiB
  constexpr bool TBG = BIG || K >= 16;
  S.runs = TBG ? bms + 2 * nw : S.tb + K * a.L.tb_words;
  S.ctrl = S.runs + a.L.max_runs;
  S.bar = reinterpret_cast<uint64_t*>(base + a.L.off_mbar);
  const uint32_t hb = a.L.hbits, B = 1u << hb, fb = a.L.fbits;  // NS == a.L.nsplit
  const uint32_t lt = lanemask_lt();
  const uint32_t tid = k * 32 + lane;
  // per-group global scratch, reused chunk after chunk (stays in L2): (d-1) of
  // recorded matches, read back only at the final match starts; big chunks:
  // then the K token-start bitmaps
  uint8_t* gscr = a.scratch + ((size_t)blockIdx.x * (blockDim.x / (32 * K)) + g) *
                                 (TBG ? enc_scratch_per_group(a.L, a.C) : 2 * (size_t)a.C);
  uint16_t* d1 = reinterpret_cast<uint16_t*>(gscr);
  if (TBG) S.tb = reinterpret_cast<uint32_t*>(gscr + 2 * (size_t)a.C);

  if (k == 0 && lane == 0) {
    mbar_init(S.bar, 1);
    fence_mbar_init();
  }
  uint32_t phase = 0;
  uint32_t next_c = 0;  // leader: prefetched next chunk index (atomic latency hidden)
  if (k == 0 && lane == 0) next_c = atomicAdd(a.counter, 1u);
#ifdef LZR_PHASE_TIMING
  long long t_ph = clock64();
#endif

  for (;;) {
    // ---- next chunk; all prior generic accesses to `data` before the TMA write
    if (k == 0 && lane == 0) {
      S.ctrl[kCtrlChunk] = next_c;
      next_c = atomicAdd(a.counter, 1u);
    }
    fence_proxy_async_smem();
    GSYNC(0);
    const uint32_t c = S.ctrl[kCtrlChunk];
    if (c >= a.N) break;
    const size_t lo = (size_t)c * a.C;
    const uint32_t n = (uint32_t)min((size_t)a.C, a.n_bytes - lo);
    const uint8_t* src = a.in + lo;
    const uint32_t P = n >= a.m ? n - a.m + 1 : 0;  // positions that can start a match
    // scatter split j covers positions [j*SS, (j+1)*SS) (SS a multiple of 32)
    const uint32_t SS = align_up((P + NS - 1) / NS, 32);
    uint8_t* out = a.slots + (size_t)c * a.C;  // the chunk's workspace slot (its stream)

    // ---- a2: stage (TMA bulk for the 16-byte multiple, LDG for the tail); zero
    //      the pre-filter, histogram and counters meanwhile
    const uint32_t n16 = n & ~15u;
    if (k == 0 && lane == 0 && n16) {
      mbar_arrive_expect_tx(S.bar, n16);
      tma_bulk_g2s(S.data, src, n16, S.bar);
    }
    for (uint32_t i = n16 + tid; i < n; i += nthr) S.data[i] = src[i];
    for (uint32_t i = n + tid; i < n + 20; i += nthr) S.data[i] = 0;
    uint32_t* hist = reinterpret_cast<uint32_t*>(S.slot);    // NS x B u16 counters
    uint32_t* seen = reinterpret_cast<uint32_t*>(S.sorted);  // 2^fb-bit filter
    for (uint32_t i = tid; i < NS * B / 2; i += nthr) hist[i] = 0;
    for (uint32_t i = tid; i < (1u << (fb - 5)); i += nthr) seen[i] = 0;
    if (tid == 0) {
      S.ctrl[kCtrlU] = 0;
      S.ctrl[kCtrlRuns] = 0;
    }
#if LZR_SKIPB
    // blocks of 32 positions whose keys are all one repeated-byte key (set by
    // the histogram pass; the scatter skips them when such keys are not indexed)
    uint32_t* skipw = S.ctrl + kCtrlProg + 2 * K;
    for (uint32_t i = tid; i < ((a.C + 1023u) >> 10); i += nthr) skipw[i] = 0;
#endif
    if (n16) {
      mbar_wait_parity(S.bar, phase);
      phase ^= 1u;
    }
    GSYNC(1);

    // ---- histogram of bucket sizes + "key hash seen before" count + run starts.
    // Raw pre-filter (sound): a match of length l at s makes s..s+l-k positions
    // with a same-key earlier occurrence, disjoint across matches; with
    // X = sum(l-3) and T tokens, S = n - X + ceil(T/8) and T >= n - 3X (m >= 4)
    // or n - 2(X + #matches) (m = 3), so S >= n whenever 11 * U <= n, U = number
    // of positions whose key hash was seen before (>= that position count).
    {
      uint32_t u = 0;
      for (uint32_t p0 = k * 32; p0 < P; p0 += nthr) {
        const uint32_t p = p0 + lane;
        bool dup = false, rs = false;
        const uint32_t key = p < P ? ld32u(S.data, p) & a.kmask : 0u;
        // 32 equal keys (a run): one atomic each instead of 32 on one address
        const uint32_t key0 = __shfl_sync(kFull, key, 0);
        const bool uni = __all_sync(kFull, p < P && key == key0);
        const uint32_t h = khash(key, hb, a.kmask);
        const uint32_t hs = (NS > 1 ? (p0 / SS) * B : 0u) + h;  // (split, bucket) counter
        const uint32_t gg = (key * 0x85EBCA6Bu) >> (32 - fb);
        if (uni) {
          uint32_t old = 0;
          if (lane == 0) {
            atomicAdd(&hist[hs >> 1], 32u << ((hs & 1u) << 4));
            old = atomicOr(&seen[gg >> 5], 1u << (gg & 31u));
#if LZR_SKIPB
            if (((key ^ (key >> 8)) & (a.kmask >> 8)) == 0) atomicOr(&skipw[p0 >> 10], 1u << ((p0 >> 5) & 31u));
#endif
          }
          old = __shfl_sync(kFull, old, 0);
          dup = lane ? true : (old & (1u << (gg & 31u))) != 0;
        } else if (p < P) {
          atomicAdd(&hist[hs >> 1], 1u << ((hs & 1u) << 4));
          dup = atomicOr(&seen[gg >> 5], 1u << (gg & 31u)) & (1u << (gg & 31u));
        }
        if (p < P)
          rs = ((key ^ (key >> 8)) & (a.kmask >> 8)) == 0 && (p == 0 || S.data[p - 1] != S.data[p]);
        u += __popc(__ballot_sync(kFull, dup));
        const uint32_t rb = __ballot_sync(kFull, rs);
        if (rb) {
          uint32_t b0 = 0;
          if (lane == 0) b0 = atomicAdd(&S.ctrl[kCtrlRuns], (uint32_t)__popc(rb));
          b0 = __shfl_sync(kFull, b0, 0);
          const uint32_t idx = b0 + __popc(rb & lt);
          if (rs && idx < a.L.max_runs) S.runs[idx] = p;
        }
      }
      if (lane == 0 && u) atomicAdd(&S.ctrl[kCtrlU], u);
    }
    GSYNC(2);
    if (11u * S.ctrl[kCtrlU] <= n) {  // certainly raw
      if (tid == 0) a.sizes[c] = n;
      continue;
    }
    const uint32_t nruns = S.ctrl[kCtrlRuns];
    // Positions whose key is one repeated byte are searched by the run-aware
    // search only (best_match_runs) when every run fits the run list and every
    // position's whole prefix is in the window; then they need no index entry:
    // their private buckets (< 256) are left empty and their candidate bits come
    // from the run structure (below).  Zero-run chunks skip most of the scatter.
    const bool skipr = hb >= 10 && nruns <= a.L.max_runs && a.W + 1 >= n;

    // ---- warp 0: exclusive scan of the B bucket totals (2 buckets per lane and
    //      round); split j's cursor of bucket h = start of h + counts of h in
    //      splits < j.  The other warps: zero the bitmaps, byte-change bitmap,
    //      walk state
#ifndef LZR_PAR_SCAN
#define LZR_PAR_SCAN 1
#endif
#ifndef LZR_PAR_SCAN8
#define LZR_PAR_SCAN8 1
#endif
// blocks of 32 positions per scatter round (their MATCH.ANY latencies
// overlap): 8 at K = 4 (mix/text/zero-runs 53.1/28.8/83.5 -> 53.9/29.2/80.3;
// 2 blocks: 52.1), 4 at K = 8 (8 KiB mix 42.6 vs 42.0 with 8) and in the lazy
// kernel (38.4 vs 37.2 with 8)
#ifndef LZR_SCATTER_BLOCKS
#define LZR_SCATTER_BLOCKS (K == 4 && !LZ ? 8 : 4)
#endif
    // K = 4 (C <= 4 KiB): the bucket scan is shared by the four warps -- each
    // scans a quarter with a local carry, then adds the totals of the quarters
    // before it -- instead of warp 0 alone while the others wait at the barrier
    // (greedy only: in the lazy kernel the same change measured 38.5 -> 35.9
    // GB/s mix -- a different register allocation of its longer walk)
    constexpr bool kParScan = LZR_PAR_SCAN && (K == 4 || (K >= 8 && LZR_PAR_SCAN8)) && NS + 2 <= K && !LZ;
    if (kParScan && (B / 2) % (32 * K) == 0) {
      const uint32_t q0 = k * (B / 2 / K), q1 = q0 + B / 2 / K;
      uint32_t carry = 0;
      for (uint32_t w0 = q0; w0 < q1; w0 += 32) {
        const uint32_t wi = w0 + lane;
        const bool priv = skipr && wi < 128;  // buckets 2w, 2w+1 < 256: left empty
        uint32_t c0 = 0, c1 = 0;  // totals of buckets 2w, 2w+1 over the splits
        for (uint32_t j = 0; j < NS; ++j) {
          const uint32_t wv = priv ? 0u : hist[j * (B / 2) + wi];
          c0 += wv & 0xFFFFu;
          c1 += wv >> 16;
        }
        const uint32_t sum = c0 + c1;
        uint32_t incl = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t t = __shfl_up_sync(kFull, incl, o);
          if ((int)lane >= o) incl += t;
        }
        uint32_t e0 = incl - sum + carry, e1 = e0 + c0;  // split j's cursors: + splits < j
        for (uint32_t j = 0; j < NS; ++j) {
          const uint32_t wv = priv ? 0u : hist[j * (B / 2) + wi];
          hist[j * (B / 2) + wi] = (e0 & 0xFFFFu) | (e1 << 16);
          e0 += wv & 0xFFFFu;
          e1 += wv >> 16;
        }
        carry += __shfl_sync(kFull, incl, 31);
      }
      if (lane == 0) S.ctrl[kCtrlProg + k] = carry;  // quarter total (prog is set up below)
      // (zeroing and the byte-change bitmap run during warp 0's scatter, below)
      GSYNC(14);
      uint32_t base = 0, all = 0;
      for (uint32_t j = 0; j < K; ++j) {
        const uint32_t t = S.ctrl[kCtrlProg + j];
        base += j < k ? t : 0u;
        all += t;
      }
      if (base)
        for (uint32_t j = 0; j < NS; ++j)
          for (uint32_t wi = q0 + lane; wi < q1; wi += 32) hist[j * (B / 2) + wi] += base | (base << 16);
      if (k == 0 && lane == 0) S.ctrl[kCtrlIdx] = all;  // index entries
      // (prog / sync are set up after the next barrier, once every warp has
      // read the quarter totals: by the last warp, with the run ends)
    } else {
    const uint32_t kk = K == 1 ? 0 : k - 1, KK = K == 1 ? 1 : K - 1;  // helper warp index
      if (k == 0) {
        uint32_t carry = 0;
        for (uint32_t w0 = 0; w0 < B / 2; w0 += 32) {
          const bool act = w0 + lane < B / 2;
          const bool priv = skipr && w0 + lane < 128;  // buckets 2w, 2w+1 < 256: left empty
          uint32_t c0 = 0, c1 = 0;  // totals of buckets 2w, 2w+1
          for (uint32_t j = 0; j < NS; ++j) {
            const uint32_t wv = act && !priv ? hist[j * (B / 2) + w0 + lane] : 0;
            c0 += wv & 0xFFFFu;
            c1 += wv >> 16;
          }
          const uint32_t sum = c0 + c1;
          uint32_t incl = sum;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(kFull, incl, o);
            if ((int)lane >= o) incl += t;
          }
          uint32_t e0 = incl - sum + carry, e1 = e0 + c0;  // running cursors
          if (act) {
            for (uint32_t j = 0; j < NS; ++j) {
              const uint32_t wv = priv ? 0u : hist[j * (B / 2) + w0 + lane];
              hist[j * (B / 2) + w0 + lane] = (e0 & 0xFFFFu) | (e1 << 16);
              e0 += wv & 0xFFFFu;
              e1 += wv >> 16;
            }
          }
          carry += __shfl_sync(kFull, incl, 31);
        }
        if (lane == 0) S.ctrl[kCtrlIdx] = carry;  // index entries (P, or fewer when skipr)
      }
      if (K == 1 || k != 0) {
        for (uint32_t i = kk * 32 + lane; i < nw; i += KK * 32) S.cand[i] = 0;
        for (uint32_t i = kk * 32 + lane; i < K * a.L.tb_words; i += KK * 32) S.tb[i] = 0;
        for (uint32_t w = kk; w < nw; w += KK) {  // change bitmap
          const uint32_t i = (w << 5) + lane;
          const bool ch = (i == 0) || (i >= n) || (S.data[i] != S.data[i - 1]);
          const uint32_t b = __ballot_sync(kFull, ch);
          if (lane == 0) S.cb[w] = b;
        }
        if (kk == 0 && lane < K) {
          S.ctrl[kCtrlProg + lane] = 0;      // prog
          S.ctrl[kCtrlProg + K + lane] = n;  // sync
        }
      }
    }
    GSYNC(3);

    // ---- warps j < NS: stable scatter of split j (positions [j*SS, (j+1)*SS))
    //      with its own cursors, 4 blocks of 32 positions per round so that the
    //      MATCH.ANY latencies overlap; the last warp then: run ends.  (A
    //      bucket-partitioned variant -- every warp scans all positions and
    //      scatters its own buckets -- measured slower: 50.1 -> 44.6 GB/s mix.)
#if LZR_SKIPB
    bool skipb = false;
    if (skipr) {
      uint32_t any = 0;
      for (uint32_t i = 0; i < ((P + 1023u) >> 10); ++i) any |= skipw[i];
      skipb = any != 0;
    }
    if (k < NS && skipb) {
      // chunks with whole blocks of not-indexed repeated-byte keys (zero runs):
      // only the other blocks, in ascending order (32 block flags per ballot)
      uint16_t* cur = S.slot + k * B;
      const uint32_t pe = min(P, (k + 1) * SS);
      const uint32_t be = (pe + 31u) >> 5;
      for (uint32_t bb = (k * SS) >> 5; bb < be; bb += 32) {
        const uint32_t myb = bb + lane;
        uint32_t lm = __ballot_sync(kFull, myb < be && !((skipw[myb >> 5] >> (myb & 31u)) & 1u));
        while (lm) {
          uint32_t h[LZR_SCATTER_BLOCKS], peers[LZR_SCATTER_BLOCKS];
          uint32_t lm2 = lm;
#pragma unroll
          for (int u = 0; u < LZR_SCATTER_BLOCKS; ++u) {
            const bool live = lm != 0;
            const uint32_t p = ((bb + (live ? (uint32_t)(__ffs(lm) - 1) : 0u)) << 5) + lane;
            lm &= lm - 1u;
            h[u] = live && p < pe ? khash(ld32u(S.data, p) & a.kmask, hb, a.kmask) : 0xFFFFFFFFu;
            if (h[u] < 256u) h[u] = 0xFFFFFFFFu;  // not indexed
          }
#pragma unroll
          for (int u = 0; u < LZR_SCATTER_BLOCKS; ++u) peers[u] = __match_any_sync(kFull, h[u]);
#pragma unroll
          for (int u = 0; u < LZR_SCATTER_BLOCKS; ++u) {
            const bool act = h[u] != 0xFFFFFFFFu;
            const uint32_t pu = ((bb + (lm2 ? (uint32_t)(__ffs(lm2) - 1) : 0u)) << 5) + lane;
            lm2 &= lm2 - 1u;
            const uint32_t basev = act ? cur[h[u]] : 0;
            if (act) S.sorted[basev + __popc(peers[u] & lt)] = (uint16_t)pu;
            __syncwarp();
            if (act && lane == 31u - __clz(peers[u])) cur[h[u]] = (uint16_t)(basev + __popc(peers[u]));
            __syncwarp();
          }
        }
      }
    } else
#endif
    if (k < NS) {
      uint16_t* cur = S.slot + k * B;
      const uint32_t pe = min(P, (k + 1) * SS);
      for (uint32_t p0 = k * SS; p0 < pe; p0 += 32 * LZR_SCATTER_BLOCKS) {
        uint32_t h[LZR_SCATTER_BLOCKS], peers[LZR_SCATTER_BLOCKS];
#pragma unroll
        for (int u = 0; u < LZR_SCATTER_BLOCKS; ++u) {
          const uint32_t p = p0 + 32 * u + lane;
          h[u] = p < pe ? khash(ld32u(S.data, p) & a.kmask, hb, a.kmask) : 0xFFFFFFFFu;
          if (skipr && h[u] < 256u) h[u] = 0xFFFFFFFFu;  // not indexed
        }
#pragma unroll
        for (int u = 0; u < LZR_SCATTER_BLOCKS; ++u) peers[u] = __match_any_sync(kFull, h[u]);
#pragma unroll
        for (int u = 0; u < LZR_SCATTER_BLOCKS; ++u) {
          const bool act = h[u] != 0xFFFFFFFFu;
          const uint32_t basev = act ? cur[h[u]] : 0;
          if (act) S.sorted[basev + __popc(peers[u] & lt)] = (uint16_t)(p0 + 32 * u + lane);
          __syncwarp();
          if (act && lane == 31u - __clz(peers[u])) cur[h[u]] = (uint16_t)(basev + __popc(peers[u]));
          __syncwarp();
        }
      }
    }
    if (kParScan && (B / 2) % (32 * K) == 0 && k >= NS) {
      // while warps < NS scatter: warps NS .. K-2 zero the bitmaps, the last
      // warp builds the byte-change bitmap (its run ends below need it)
      constexpr uint32_t kZ = K > NS + 1 ? K - 1 - NS : 1;  // zeroing warps
      if (k + 1 < K) {
        for (uint32_t i = (k - NS) * 32 + lane; i < nw; i += kZ * 32) S.cand[i] = 0;
        for (uint32_t i = (k - NS) * 32 + lane; i < K * a.L.tb_words; i += kZ * 32) S.tb[i] = 0;
      } else {
        for (uint32_t w = 0; w < nw; ++w) {
          const uint32_t i = (w << 5) + lane;
          const bool ch = (i == 0) || (i >= n) || (S.data[i] != S.data[i - 1]);
          const uint32_t b = __ballot_sync(kFull, ch);
          if (lane == 0) S.cb[w] = b;
        }
        __syncwarp();
      }
    }
    if (k == K - 1) {
      if (kParScan && (B / 2) % (32 * K) == 0 && lane < K) {
        S.ctrl[kCtrlProg + lane] = 0;      // prog
        S.ctrl[kCtrlProg + K + lane] = n;  // sync
      }
      for (uint32_t j = lane; j < min(nruns, a.L.max_runs); j += 32) {
        const uint32_t st = S.runs[j];
        S.runs[j] = ((st + run_len(S.cb, st, n - st) - 1u) << 16) | st;  // (end - 1, start): 16 bits each
      }
    }
    GSYNC(4);

    // ---- mark the first entry of every non-empty bucket (the last split's
    //      cursor of h = end of h)
    if (!BIG) {  // (big chunks: bucket ends instead of marks)
      const uint16_t* endc = S.slot + (NS - 1) * B;
      for (uint32_t hh = tid; hh < B; hh += nthr) {
        const uint32_t st = hh ? endc[hh - 1] : 0u;
        if (endc[hh] > st) S.sorted[st] |= kFirst;
      }
    }
    GSYNC(5);

    // ---- slot of each position and the candidate bitmap: the nearest same-key
    //      earlier position is the nearest same-key entry below in the bucket
    const uint32_t nidx = S.ctrl[kCtrlIdx];
    for (uint32_t sl = tid; sl < nidx && !BIG; sl += nthr) {
      const uint32_t e = S.sorted[sl];
      const uint32_t q = e & kPos;
      S.slot[q] = (uint16_t)sl;
      if (!(e & kFirst)) {
        const uint32_t kq = ld32u(S.data, q) & a.kmask;
        bool has = false;
        for (uint32_t s2 = sl - 1;; --s2) {
          const uint32_t e2 = S.sorted[s2];
          const uint32_t q2 = e2 & kPos;
          if ((ld32u(S.data, q2) & a.kmask) == kq) {
            has = q - q2 <= a.W;
            break;
          }
          if (e2 & kFirst) break;
        }
        if (has) atomicOr(&S.cand[q >> 5], 1u << (q & 31u));
      }
    }
    for (uint32_t sl = tid; sl < nidx && BIG; sl += nthr) {
      // big chunks: the bucket's first entry from the bucket ends
      const uint32_t q = S.sorted[sl];
      const uint32_t kq = ld32u(S.data, q) & a.kmask;
      const uint32_t h = khash(kq, hb, a.kmask);
      const uint32_t bs = h ? S.slot[(NS - 1) * B + h - 1] : 0u;
      bool has = false;
      for (uint32_t s2 = sl; s2 > bs;) {
        const uint32_t q2 = S.sorted[--s2];
        if ((ld32u(S.data, q2) & a.kmask) == kq) {
          has = q - q2 <= a.W;
          break;
        }
      }
      if (has) atomicOr(&S.cand[q >> 5], 1u << (q & 31u));
    }
    if (skipr && nruns) {
      // not-indexed positions (key = k copies of one byte): inside a run (the
      // byte before is the same) the key also occurs at d = 1; a run start has a
      // candidate iff an earlier run of the same byte (length >= k) exists
      for (uint32_t w = tid; w < (P + 31) >> 5; w += nthr) {
        const uint32_t c0 = S.cb[w], c1 = S.cb[w + 1];
        uint32_t z = c0;  // cb bit p (byte p differs from p-1) ...
        for (uint32_t j = 1; j < a.kbytes; ++j) z |= __funnelshift_r(c0, c1, j);  // ... or p+1..p+k-1
        const uint32_t mrun = ~z & valid_mask(P, w);
        if (mrun) atomicOr(&S.cand[w], mrun);
      }
      if (k == 0) {
        for (uint32_t j = lane; j < nruns; j += 32) {
          const uint32_t st = S.runs[j] & 0xFFFFu, b = S.data[st];
          bool has = false;
          for (uint32_t i = 0; i < nruns && !has; ++i) {
            const uint32_t t = S.runs[i] & 0xFFFFu;
            has = t < st && S.data[t] == b;
          }
          if (has && st < P) atomicOr(&S.cand[st >> 5], 1u << (st & 31u));
        }
      }
    }
    GSYNC(6);

    // ---- a3/a4: the K speculative walk segments
    {
      // later positions have more candidates: segment bounds balance a work
      // density growing ~linearly with the position (walk_bound)
      // up to 4 KiB (K <= 4): bounds from the candidate bitmap; above, the work
      // per candidate grows along the chunk (longer lists), which the fixed
      // slope models better (C = 8/16/32 KiB mix: 41.4/23.9/11.1 GB/s with the
      // slope vs 41.1/23.5/10.8 with candidate weights)
      uint32_t start, nb;
      if (K <= 4 && LZR_WALK_CAND_A + 0 > 0) {
        const uint32_t nwords = (n + 31) >> 5;
        uint32_t tot = 0;
        for (uint32_t w0 = 0; w0 < nwords; w0 += 32) {
          const uint32_t w = w0 + lane;
          tot += __reduce_add_sync(kFull, w < nwords ? LZR_WALK_CAND_A * __popc(S.cand[w]) + LZR_WALK_CAND_B : 0u);
        }
        start = walk_bound_cand(S.cand, nwords, n, k, K, tot, lane);
        nb = walk_bound_cand(S.cand, nwords, n, k + 1, K, tot, lane);
      } else {
        start = walk_bound(n, k, K);
        nb = walk_bound(n, k + 1, K);
      }
      if (start < n && (k == 0 || start > 0))
        walk_segment<K, LZ, BIG, TBG>(S, d1, k, start, nb, n, P, nruns, a, lane);
    }
    GSYNC(7);

    // ---- final token-start bitmap = chain warp 0 -> warp 1 -> ... through the
    //      meeting points (into the dead candidate bitmap); zero the
    //      token-index match bitmap (dead byte-change bitmap)
    for (uint32_t i = tid; i < nw; i += nthr) {
      S.cand[i] = 0;
      S.cb[i] = 0;
    }
    GSYNC(8);
    {
      uint32_t lo_k = 0, hi_k = 0;
      bool in_chain = false;
      uint32_t x = 0;
      for (uint32_t w = 0; w < K; ++w) {
        const uint32_t y = S.ctrl[kCtrlProg + K + w];
        if (w == k) {
          in_chain = true;
          lo_k = x;
          hi_k = y;
        }
        if (y >= n) break;
        x = y;
      }
      if (in_chain && lo_k < hi_k) {
        const uint32_t* tbk = S.tb + k * a.L.tb_words;
        for (uint32_t w = (lo_k >> 5) + lane; w <= (hi_k - 1) >> 5; w += 32) {
          uint32_t b = tbk[w];
          const uint32_t wlo = w << 5;
          if (wlo < lo_k) b &= 0xFFFFFFFFu << (lo_k - wlo);
          if (hi_k - wlo < 32) b &= (1u << (hi_k - wlo)) - 1u;
          if (b) atomicOr(&S.cand[w], b);
        }
      }
      if (tid == 0) atomicOr(&S.cand[n >> 5], 1u << (n & 31u));  // sentinel: a token "starts" at n
    }
    GSYNC(9);

    // ---- a5: totals.  A token at p is a match iff no token starts at p + 1.
    const uint32_t nwords = (n + 31) >> 5;
    const uint32_t w_lo = (nwords * k) / K, w_hi = (nwords * (k + 1)) / K;
    {
      uint32_t T = 0, M = 0;
      for (uint32_t w = w_lo + lane; w < w_hi; w += 32) {
        const uint32_t cw = S.cand[w];
        const uint32_t t = cw & valid_mask(n, w);
        const uint32_t mm = t & ~((cw >> 1) | (S.cand[w + 1] << 31));
        T += __popc(t);
        M += __popc(mm);
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        T += __shfl_xor_sync(kFull, T, o);
        M += __shfl_xor_sync(kFull, M, o);
      }
      if (lane == 0) {
        S.ctrl[kCtrlProg + k] = T;
        S.ctrl[kCtrlProg + K + k] = M;
      }
    }
    GSYNC(10);
    uint32_t Ttot = 0, Mtot = 0, Tb = 0, Mb = 0;
    for (uint32_t w = 0; w < K; ++w) {
      const uint32_t t = S.ctrl[kCtrlProg + w], m = S.ctrl[kCtrlProg + K + w];
      if (w < k) {
        Tb += t;
        Mb += m;
      }
      Ttot += t;
      Mtot += m;
    }
    const uint32_t Sz = Ttot + 2 * Mtot + ((Ttot + 7) >> 3);
    if (Sz >= n) {  // not shorter than the chunk: stored raw (R9)
      if (tid == 0) a.sizes[c] = n;
      continue;
    }

    // ---- pass 0: match bit per token index (source of the flag bytes);
    //      pass 1: every token's bytes.  The warp's words in rounds of 32:
    //      lane-parallel counts + scan give each word's token/match bases.
    uint8_t* ob = reinterpret_cast<uint8_t*>(S.sorted);  // the index is dead now
    for (int pass = 0; pass < 2; ++pass) {
      uint32_t tb_run = Tb, mb_run = Mb;
      for (uint32_t w0 = w_lo; w0 < w_hi; w0 += 32) {
        const uint32_t w = w0 + lane;
        uint32_t t = 0, mm = 0;
        if (w < w_hi) {
          const uint32_t cw = S.cand[w];
          t = cw & valid_mask(n, w);
          mm = t & ~((cw >> 1) | (S.cand[w + 1] << 31));
        }
        const uint32_t pt = __popc(t), pm = __popc(mm);
        uint32_t ti = pt, mi = pm;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t a1 = __shfl_up_sync(kFull, ti, o), b1 = __shfl_up_sync(kFull, mi, o);
          if ((int)lane >= o) {
            ti += a1;
            mi += b1;
          }
        }
        const uint32_t tbase = tb_run + ti - pt, mbase = mb_run + mi - pm;
        tb_run += __shfl_sync(kFull, ti, 31);
        mb_run += __shfl_sync(kFull, mi, 31);
        if (pass == 0) {
          uint32_t rem = mm;  // this lane's word: token indices of its matches
          while (rem) {
            const uint32_t bit = (uint32_t)(__ffs(rem) - 1);
            rem &= rem - 1;
            const uint32_t j = tbase + __popc(t & ((1u << bit) - 1u));
            atomicOr(&S.cb[j >> 5], 1u << (j & 31u));
            const uint32_t pm = (w << 5) + bit;
            if (!BIG) S.slot[pm] = __ldcg(d1 + pm);  // the slot array is dead after the walk
          }
        } else {
          const uint32_t nwr = min(32u, w_hi - w0);
          for (uint32_t i = 0; i < nwr; ++i) {
            const uint32_t tw = __shfl_sync(kFull, t, i), mw = __shfl_sync(kFull, mm, i);
            const uint32_t tbw = __shfl_sync(kFull, tbase, i), mbw = __shfl_sync(kFull, mbase, i);
            if ((tw >> lane) & 1u) {
              const uint32_t p = ((w0 + i) << 5) + lane;
              const uint32_t j = tbw + __popc(tw & lt);
              const uint32_t mbef = mbw + __popc(mw & lt);
              const uint32_t pos = j + 2 * mbef + (j >> 3) + 1;
              if ((j & 7u) == 0) ob[pos - 1] = (uint8_t)(S.cb[j >> 5] >> (j & 24u));
              if ((mw >> lane) & 1u) {
                // length = distance to the next token start (sentinel at n)
                uint32_t ww = (p + 1) >> 5;
                uint32_t b = S.cand[ww] & (0xFFFFFFFFu << ((p + 1) & 31u));
                while (!b) b = S.cand[++ww];
                const uint32_t l = (ww << 5) + (uint32_t)(__ffs(b) - 1) - p;
                const uint32_t dm1 = BIG ? (uint32_t)__ldcg(d1 + p) : (uint32_t)S.slot[p];
                ob[pos] = (uint8_t)(dm1 & 0xFF);
                ob[pos + 1] = (uint8_t)(dm1 >> 8);
                ob[pos + 2] = (uint8_t)(l - a.m);
              } else {
                ob[pos] = S.data[p];
              }
            }
          }
        }
      }
      GSYNC(11);
    }

    // ---- copy the staged stream to the chunk's workspace slot (16-byte stores;
    //      every d1 read happened before the last group barrier)
    const uint32_t n16o = align_up(Sz, 16);
    const uint32_t* ob32 = reinterpret_cast<const uint32_t*>(ob);  // staging is 4-byte aligned
    for (uint32_t i = tid * 16; i < n16o; i += nthr * 16)
      *reinterpret_cast<uint4*>(out + i) =
          make_uint4(ob32[i >> 2], ob32[(i >> 2) + 1], ob32[(i >> 2) + 2], ob32[(i >> 2) + 3]);
    if (tid == 0) a.sizes[c] = Sz;
  }
}

template <int K, int NS, bool LZ, bool G1 = false, bool BIG = false, uint32_t CF = 0, bool DEF = false>
cudaError_t launch_k(const EncArgs& a, int sm_count, int smem_optin, cudaStream_t s, int* launches) {
  int groups = smem_optin / (int)a.L.per_group;
  const int max_groups = MaxThreads<K, G1>::value / (32 * K);
  if (groups > max_groups) groups = max_groups;
  if (groups > 15) groups = 15;  // named barriers 1..15
  if (groups < 1) return cudaErrorInvalidConfiguration;
  const size_t smem = (size_t)groups * a.L.per_group;
  // Host calls cached per device so that batch-by-batch callers (the host
  // pipeline) do not pay them on every launch.  The dynamic shared-memory limit
  // of this instantiation is raised once to the device's opt-in maximum and
  // never lowered, so concurrent callers with different chunk sizes cannot
  // undercut each other's launch; the occupancy is cached per smem size.
  struct Cached {
    bool attr;
    size_t smem;
    int per_sm;
  };
  static Cached cache[64] = {};
  static std::mutex mu;
  int dev = 0;
  cudaError_t err = cudaGetDevice(&dev);
  if (err != cudaSuccess) return err;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  int per_sm = 0;
  {
    std::lock_guard<std::mutex> lk(mu);
    if (!cache[dev].attr) {
      err = cudaFuncSetAttribute(lzr_encode_kernel<K, NS, LZ, G1, BIG, CF, DEF>,
                                 cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin);
      if (err != cudaSuccess) return err;
      cache[dev].attr = true;
    }
    if (cache[dev].smem == smem) per_sm = cache[dev].per_sm;
  }
  if (per_sm == 0) {
    // persistent grid: every resident CTA (one per SM unless MinBlocks > 1)
    per_sm = 1;
    if (MinBlocks<K, G1, BIG>::value > 1 &&
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lzr_encode_kernel<K, NS, LZ, G1, BIG, CF, DEF>,
                                                      groups * 32 * K, smem) != cudaSuccess)
      per_sm = 1;
    if (per_sm < 1) per_sm = 1;
    std::lock_guard<std::mutex> lk(mu);
    cache[dev].smem = smem;
    cache[dev].per_sm = per_sm;
  }
  const uint32_t need = (a.N + groups - 1) / groups;
  const uint32_t cap = (uint32_t)(sm_count * per_sm);
  const uint32_t grid = need < cap ? need : cap;
  lzr_encode_kernel<K, NS, LZ, G1, BIG, CF, DEF><<<grid, groups * 32 * K, smem, s>>>(a);
  if (launches) ++*launches;
  return cudaGetLastError();
}

}  // namespace

#ifdef LZR_PHASE_TIMING
extern "C" int lzr_debug_phase_times(unsigned long long* out) {
  if (cudaMemcpyFromSymbol(out, g_phase, sizeof(g_phase)) != cudaSuccess) return -4;
  static unsigned long long zero[16][4][2];
  return cudaMemcpyToSymbol(g_phase, zero, sizeof(g_phase)) == cudaSuccess ? 0 : -4;
}
#endif

namespace {
// the instantiation specialised for chunk size CF and the configs' parameters
// (W = C, m = 4, M = 259) when the call has them, else the generic one
template <int K, int NS, bool LZ, bool BIG, uint32_t CF>
cudaError_t launch_cf(const EncArgs& a, int sm_count, int smem_optin, cudaStream_t s, int* launches) {
  if (a.C == CF && a.W == CF && a.m == 4 && a.M == 259)
    return launch_k<K, NS, LZ, false, BIG, CF, true>(a, sm_count, smem_optin, s, launches);
  return launch_k<K, NS, LZ, false, BIG>(a, sm_count, smem_optin, s, launches);
}

template <bool LZ>
cudaError_t launch_kns(const EncArgs& a, int sm_count, int smem_optin, cudaStream_t s, int* launches) {
  switch (a.L.K) {
    case 1: return launch_k<1, 1, LZ>(a, sm_count, smem_optin, s, launches);
    case 2: return launch_k<2, 1, LZ>(a, sm_count, smem_optin, s, launches);
    case 3: return launch_k<3, 1, LZ>(a, sm_count, smem_optin, s, launches);
    case 4:
      switch (a.L.nsplit) {
        case 1:
          // few waves of chunks: one group per CTA (see MaxThreads)
          if (a.C == 4096 && a.W == 4096 && a.m == 4 && a.M == 259) {  // the configs' parameters
            if (a.N < kG1MaxWaves * 9u * (uint32_t)sm_count)
              return launch_k<4, 1, LZ, true, false, 4096, true>(a, sm_count, smem_optin, s, launches);
            return launch_k<4, 1, LZ, false, false, 4096, true>(a, sm_count, smem_optin, s, launches);
          }
          if (a.N < kG1MaxWaves * 9u * (uint32_t)sm_count)
            return a.C == 4096 ? launch_k<4, 1, LZ, true, false, 4096>(a, sm_count, smem_optin, s, launches)
                               : launch_k<4, 1, LZ, true>(a, sm_count, smem_optin, s, launches);
          return a.C == 4096 ? launch_k<4, 1, LZ, false, false, 4096>(a, sm_count, smem_optin, s, launches)
                             : launch_k<4, 1, LZ>(a, sm_count, smem_optin, s, launches);
        case 2: return launch_k<4, 2, LZ>(a, sm_count, smem_optin, s, launches);
        case 4: return launch_k<4, 4, LZ>(a, sm_count, smem_optin, s, launches);
        default: return cudaErrorInvalidConfiguration;
      }
    case 32:  // chunks above 16 KiB: one group of 32 warps per SM
      if (enc_big(a.C)) {
        if (a.L.nsplit != 2) return cudaErrorInvalidConfiguration;
        // (not specialised: 64 KiB measured 16.2 specialised vs 16.6 generic)
        return launch_k<32, 2, LZ, false, true>(a, sm_count, smem_optin, s, launches);
      }
      if (a.L.nsplit != 4) return cudaErrorInvalidConfiguration;
      return launch_cf<32, 4, LZ, false, 32768>(a, sm_count, smem_optin, s, launches);
    case 16:  // 8 KiB < C <= 16 KiB: groups of 16 warps, two per SM
#if LZR_BIG_WARPS == 16
      if (enc_big(a.C)) {
        switch (a.L.nsplit) {
          case 1: return launch_k<16, 1, LZ, false, true>(a, sm_count, smem_optin, s, launches);
          case 2: return launch_k<16, 2, LZ, false, true>(a, sm_count, smem_optin, s, launches);
          case 4: return launch_k<16, 4, LZ, false, true>(a, sm_count, smem_optin, s, launches);
          default: return cudaErrorInvalidConfiguration;
        }
      }
#endif
      if (a.L.nsplit != 4) return cudaErrorInvalidConfiguration;
      return launch_cf<16, 4, LZ, false, 16384>(a, sm_count, smem_optin, s, launches);
    case 8:
      switch (a.L.nsplit) {
        case 1: return launch_k<8, 1, LZ>(a, sm_count, smem_optin, s, launches);
        case 2: return launch_k<8, 2, LZ>(a, sm_count, smem_optin, s, launches);
        case 4: return launch_cf<8, 4, LZ, false, 8192>(a, sm_count, smem_optin, s, launches);
        case 8: return launch_k<8, 8, LZ>(a, sm_count, smem_optin, s, launches);
        default: return cudaErrorInvalidConfiguration;
      }
    default: return cudaErrorInvalidConfiguration;
  }
}
}  // namespace

cudaError_t launch_encode(const EncArgs& a, int sm_count, int smem_optin, cudaStream_t s,
                          int* launches) {
  return a.lazy ? launch_kns<true>(a, sm_count, smem_optin, s, launches)
                : launch_kns<false>(a, sm_count, smem_optin, s, launches);
}

}  // namespace lzr
