/*
 * synth/synth_core.h -- seeded synthetic write-stream generator.
 *
 * Input generator shared by the tests, the oracle baseline and the bench.  It
 * holds none of the method's arithmetic (no matching, no encoding): it only
 * produces bytes.  The same source compiles for the host (synth_host.c, gcc)
 * and the device (synth_cuda.cu, nvcc), so both sides draw bit-identical
 * streams from a counter-based generator: chunk i of a stream depends only on
 * (seed, class, i, chunk length), never on the batch it is generated in.
 *
 * Workload recipe: the paper used
 * vdbench streams with compression ratio 2.0 (§4 "The deduplication and
 * compression ratio are set to 2.0"), which are not available.  Classes:
 *   T  text-like : words of a seeded 1024-word vocabulary (lengths 3..9,
 *                  [a-z]) drawn Zipf(s = 1.1); separators ' ' 85%, ", " 5%,
 *                  ". " 5%, '\n' 5%
 *   R  random    : uniform bytes
 *   Z  zero-runs : alternating zero runs U[16,512] and random runs U[8,64]
 *   MIX          : per-chunk class T 40% / R 30% / Z 30%
 *   CR2          : per-chunk class T 40% / R 20% / Z 40%  (tuned so the
 *                  oracle's stream ratio is ~2.0, the paper's setting)
 */
#ifndef SYNTH_CORE_H
#define SYNTH_CORE_H
#include <stdint.h>

#ifdef __CUDACC__
#define SYN_FN static __host__ __device__ __forceinline__
#else
#define SYN_FN static inline
#endif

enum { SYN_TEXT = 0, SYN_RANDOM = 1, SYN_ZERORUNS = 2, SYN_MIX = 3, SYN_CR2 = 4, SYN_NCLASS = 5 };

#define SYN_VOCAB 1024
#define SYN_WORD_MAX 9

typedef struct syn_tables {
  uint32_t cdf[SYN_VOCAB];              /* Zipf CDF scaled to 2^32, strictly increasing */
  uint8_t wlen[SYN_VOCAB];              /* 3..9 */
  uint8_t word[SYN_VOCAB][SYN_WORD_MAX + 1];
} syn_tables;

#define SYN_GOLDEN 0x9E3779B97F4A7C15ull

SYN_FN uint64_t syn_mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

/* splitmix64 stream whose start state is a function of (seed, chunk index). */
typedef struct syn_rng {
  uint64_t s;
} syn_rng;

SYN_FN syn_rng syn_chunk_rng(uint64_t seed, uint64_t chunk) {
  syn_rng r;
  r.s = syn_mix(seed ^ syn_mix(chunk + 0x5EEDull));
  return r;
}

SYN_FN uint64_t syn_next(syn_rng* r) {
  r->s += SYN_GOLDEN;
  return syn_mix(r->s);
}

/* class actually used for a chunk */
SYN_FN int syn_chunk_class(int cls, uint64_t seed, uint64_t chunk) {
  if (cls == SYN_MIX || cls == SYN_CR2) {
    uint32_t u = (uint32_t)(syn_mix(seed ^ syn_mix(chunk ^ 0xC1A55C1A55ull)) % 100u);
    if (cls == SYN_MIX) return u < 40 ? SYN_TEXT : (u < 70 ? SYN_RANDOM : SYN_ZERORUNS);
    return u < 40 ? SYN_TEXT : (u < 60 ? SYN_RANDOM : SYN_ZERORUNS);
  }
  return cls;
}

SYN_FN void syn_fill_random(uint8_t* out, uint32_t n, syn_rng* r) {
  uint32_t i = 0;
  while (i < n) {
    uint64_t v = syn_next(r);
    for (int k = 0; k < 8 && i < n; ++k, ++i) out[i] = (uint8_t)(v >> (8 * k));
  }
}

SYN_FN void syn_fill_zeroruns(uint8_t* out, uint32_t n, syn_rng* r) {
  uint32_t i = 0;
  int zero = 1;
  while (i < n) {
    uint64_t v = syn_next(r);
    uint32_t len = zero ? 16u + (uint32_t)(v % 497u) : 8u + (uint32_t)(v % 57u);
    if (len > n - i) len = n - i;
    if (zero) {
      for (uint32_t k = 0; k < len; ++k) out[i + k] = 0;
    } else {
      syn_fill_random(out + i, len, r);
    }
    i += len;
    zero = !zero;
  }
}

SYN_FN uint32_t syn_zipf_pick(const syn_tables* t, uint32_t u) {
  /* first rank whose cdf exceeds u (binary search) */
  uint32_t lo = 0, hi = SYN_VOCAB - 1;
  while (lo < hi) {
    uint32_t mid = (lo + hi) >> 1;
    if (t->cdf[mid] > u) hi = mid; else lo = mid + 1;
  }
  return lo;
}

SYN_FN void syn_fill_text(uint8_t* out, uint32_t n, syn_rng* r, const syn_tables* t) {
  uint32_t i = 0;
  while (i < n) {
    uint64_t v = syn_next(r);
    uint32_t w = syn_zipf_pick(t, (uint32_t)v);
    uint32_t L = t->wlen[w];
    for (uint32_t k = 0; k < L && i < n; ++k) out[i++] = t->word[w][k];
    uint32_t s = (uint32_t)((v >> 32) % 100u);
    if (s < 85) {
      if (i < n) out[i++] = ' ';
    } else if (s < 95) {
      if (i < n) out[i++] = (uint8_t)(s < 90 ? ',' : '.');
      if (i < n) out[i++] = ' ';
    } else {
      if (i < n) out[i++] = '\n';
    }
  }
}

/* Dedup-2.0 logical stream (config 5; §4 "The deduplication and
 * compression ratio are set to 2.0"): logical chunk i is fresh w.p. 1/2 (chunk
 * 0 always); a duplicate copies the content of the nearest fresh chunk at or
 * below a uniformly drawn earlier index r < i.  Content of a fresh chunk j = the
 * base class's chunk j, so distinct fresh chunks differ (with overwhelming
 * probability) and logical/unique ~ 2.0.  The flag SYN_DEDUP on the class
 * selects this mapping. */
#define SYN_DEDUP 0x10

SYN_FN int syn_fresh(uint64_t seed, uint64_t i) {
  return i == 0 || (syn_mix(seed ^ syn_mix(i ^ 0xDED0DED0ull)) & 1u);
}

SYN_FN uint64_t syn_dedup_source(uint64_t seed, uint64_t i) {
  if (syn_fresh(seed, i)) return i;
  uint64_t r = syn_mix(seed ^ syn_mix(i ^ 0x50C0CE5ull)) % i;
  while (!syn_fresh(seed, r)) --r;
  return r;
}

/* Generate chunk `chunk` (global index) of length n into out. */
SYN_FN void syn_fill_chunk(uint8_t* out, uint32_t n, int cls, uint64_t seed, uint64_t chunk,
                           const syn_tables* t) {
  if (cls & SYN_DEDUP) {
    cls &= ~SYN_DEDUP;
    chunk = syn_dedup_source(seed, chunk);
  }
  int c = syn_chunk_class(cls, seed, chunk);
  syn_rng r = syn_chunk_rng(seed, chunk);
  if (c == SYN_TEXT) syn_fill_text(out, n, &r, t);
  else if (c == SYN_RANDOM) syn_fill_random(out, n, &r);
  else syn_fill_zeroruns(out, n, &r);
}

#endif
