/*
 * cpuref/lzr_fast.c -- FAST EXACT CPU COMPRESSOR (TEST INFRASTRUCTURE AND CPU
 * BASELINE ONLY).
 *
 * The paper's CPU-side compression (§3.2(1) "there is no data dependency
 * between chunks, so we can run compression independently on each chunk ...
 * assigning a computing thread ... to each chunk") and the CPU arm of its
 * GPU-usage decision (§3.2(3) "we compare the compression performance of
 * the CPU and the GPU to determine when to use the GPU").  It computes exactly
 * what oracle/lzr_ref.c computes (same readings R1-R11, R21) but finds the
 * longest match through hash chains instead of an exhaustive scan, so that
 * whole multi-GiB streams can be checked chunk by chunk and the CPU baseline
 * is a fair one.  It is pinned to the plain oracle, not the other way round:
 * tests/test_cpuref.py requires byte equality with oracle/ on every stream
 * class, adversarial inputs, a parameter grid and brute force on tiny inputs.
 *
 * Only tests/, bench.py (cpu_fast / integration keys) and tools/ may load it.
 * It shares no code, header or table with the CUDA path or with oracle/.
 *
 * Search (exact):
 *   - k = min(m, 4) key bytes.  Every match of length >= m starts with the same
 *     k bytes, so the candidates of p are the earlier positions with p's key:
 *     a chain per key hash (prev[] links, ascending insertion => the chain from
 *     p walks nearest first), each entry's key re-checked (a collision may only
 *     cost time).  Walk while p - q <= W; a candidate is compared only if it
 *     also matches the byte at the current best length; stop at the cap.
 *     Strict '>' in nearest-first order = "longest, then nearest" (R6, R7).
 *   - keys of k copies of one byte b with the whole prefix inside the window:
 *     every candidate lies in a run of b.  With r = min(run length at p, cap),
 *     an earlier run [s, e) contributes its best (and nearest among equals)
 *     candidate q = e - r with length r + LCP(x[p+r..], x[e..]) (capped) when
 *     e - s >= r, else q = s with length e - s; p's own run gives d = 1 with
 *     length r.  So one comparison per earlier run replaces chains of
 *     thousands of positions in zero runs.
 */
#include "lzr_fast.h"

#include <pthread.h>
#include <stdatomic.h>
#include <stdlib.h>
#include <string.h>

int lzr_fast_validate(const lzr_fast_params* p) {
  if (!p) return -1;
  if (p->chunk_size < 16 || p->chunk_size > 65536 || (p->chunk_size % 16) != 0) return -1;
  if (p->window < 1 || p->window > p->chunk_size) return -1;
  if (p->min_match < 3 || p->min_match > 255) return -1;
  if (p->max_match < p->min_match || p->max_match > p->min_match + 255) return -1;
  if (p->tie_break != 0 || p->parse > 1) return -2;
  return 0;
}

#define HBITS 15
#define HSIZE (1u << HBITS)

typedef struct {
  const uint8_t* x;
  uint32_t n, W, m, M, k, P;
  uint32_t* head; /* [HSIZE]: (epoch << 16) | position; stale epochs = empty */
  uint32_t epoch;
  int32_t* prev; /* [n] */
  /* runs of one byte value of length >= k: start/end, linked per byte value
   * in ascending order (run_first[b] .. run_next[]) */
  uint32_t* run_s;
  uint32_t* run_e;
  int32_t* run_next;
  int32_t run_first[256];
  int32_t* run_of; /* run index of position p (-1 if not inside a run >= k) */
} chunk_ctx;

/* first k bytes at p, little-endian (the chunk buffer has 16 zero bytes of slack) */
static inline uint32_t key_at(const uint8_t* x, uint32_t p, uint32_t k) {
  uint32_t v;
  memcpy(&v, x + p, 4);
  return k == 4 ? v : (v & ((1u << (8 * k)) - 1u));
}

static inline uint32_t hash_key(uint32_t key) { return (key * 2654435761u) >> (32 - HBITS); }

static inline uint32_t lcp(const uint8_t* x, uint32_t a, uint32_t b, uint32_t lim) {
  uint32_t l = 0;
  while (l + 8 <= lim) {
    uint64_t va, vb;
    memcpy(&va, x + a + l, 8);
    memcpy(&vb, x + b + l, 8);
    if (va != vb) return l + (uint32_t)(__builtin_ctzll(va ^ vb) >> 3);
    l += 8;
  }
  while (l < lim && x[a + l] == x[b + l]) ++l;
  return l;
}

/* returns U = number of positions whose key hash occurred earlier in the chunk */
static uint32_t build(chunk_ctx* c) {
  const uint8_t* x = c->x;
  /* a new epoch per chunk empties the table without clearing it */
  if (++c->epoch == 0x10000u) {
    memset(c->head, 0, HSIZE * sizeof(uint32_t));
    c->epoch = 1;
  }
  const uint32_t ep = c->epoch << 16;
  uint32_t U = 0;
  for (uint32_t p = 0; p < c->P; ++p) {
    const uint32_t h = hash_key(key_at(x, p, c->k));
    const uint32_t e = c->head[h];
    c->prev[p] = (e & 0xFFFF0000u) == ep ? (int32_t)(e & 0xFFFFu) : -1;
    U += c->prev[p] >= 0;
    c->head[h] = ep | p;
  }
  for (int b = 0; b < 256; ++b) c->run_first[b] = -1;
  int32_t last[256];
  for (int b = 0; b < 256; ++b) last[b] = -1;
  uint32_t nr = 0, p = 0;
  while (p < c->n) {
    uint32_t e = p + 1;
    while (e < c->n && x[e] == x[p]) ++e;
    if (e - p >= c->k) {
      c->run_s[nr] = p;
      c->run_e[nr] = e;
      c->run_next[nr] = -1;
      if (last[x[p]] < 0) c->run_first[x[p]] = (int32_t)nr;
      else c->run_next[last[x[p]]] = (int32_t)nr;
      last[x[p]] = (int32_t)nr;
      for (uint32_t i = p; i < e; ++i) c->run_of[i] = (int32_t)nr;
      ++nr;
    } else {
      for (uint32_t i = p; i < e; ++i) c->run_of[i] = -1;
    }
    p = e;
  }
  return U;
}

/* best capped match at p: *len (< m: none), *dist */
static void best_match(const chunk_ctx* c, uint32_t p, uint32_t* len, uint32_t* dist) {
  *len = 0;
  *dist = 0;
  if (p >= c->P || p == 0) return;
  const uint8_t* x = c->x;
  const uint32_t cap = (c->n - p) < c->M ? (c->n - p) : c->M;
  const uint32_t kp = key_at(x, p, c->k);
  uint32_t best = 0, bq = 0;
  const int32_t ri = c->run_of[p];
  if (ri >= 0 && c->run_e[ri] - p >= c->k && p <= c->W) {
    /* run-aware (every same-key candidate lies in a run of x[p]) */
    const uint32_t s0 = c->run_s[ri], e0 = c->run_e[ri];
    const uint32_t r = (e0 - p) < cap ? (e0 - p) : cap;
    if (p > s0) {
      best = r;
      bq = p - 1;
    }
    for (int32_t j = c->run_first[x[p]]; j >= 0 && j != ri; j = c->run_next[j]) {
      const uint32_t s = c->run_s[j], e = c->run_e[j];
      uint32_t q, l;
      if (e - s >= r) {
        q = e - r;
        l = r < cap ? r + lcp(x, p + r, e, cap - r) : cap;
      } else {
        q = s;
        l = e - s;
      }
      /* longer, or equal and nearer (larger q) */
      if (l > best || (l == best && l > 0 && q > bq)) {
        best = l;
        bq = q;
      }
    }
  } else {
    for (int32_t qi = c->prev[p]; qi >= 0; qi = c->prev[qi]) {
      const uint32_t q = (uint32_t)qi;
      if (p - q > c->W) break;
      if (key_at(x, q, c->k) != kp) continue;
      if (best && x[q + best] != x[p + best]) continue;
      const uint32_t l = lcp(x, p, q, cap);
      if (l > best) {
        best = l;
        bq = q;
        if (best == cap) break;
      }
    }
  }
  if (best >= c->m) {
    *len = best;
    *dist = p - bq;
  }
}

/* parse + R1 encode + raw fallback (R9) of one chunk into out (>= n bytes) */
static uint32_t compress_chunk(chunk_ctx* c, uint32_t parse, uint8_t* out, uint8_t* tmp) {
  const uint8_t* x = c->x;
  const uint32_t n = c->n;
  /* Raw pre-check (sound, R9): a match of length l covers l - k + 1 >= l - 3
   * positions whose key occurred earlier, disjoint across matches, so with
   * X = sum(l - 3) <= U the stream needs S = n - X + ceil(T/8) bytes with
   * T >= n - 3X (m >= 4; n - 2(X + #matches) for m = 3): S >= n when 11 U <= n. */
  if (11u * build(c) <= n) {
    memcpy(out, x, n);
    return n;
  }
  uint32_t p = 0, pos = 0, ntok = 0, flag_pos = 0;
  uint32_t cl = 0, cd = 0, cp = 0xFFFFFFFFu; /* lazy: best match known at cp */
  while (p < n) {
    uint32_t l, d;
    if (p == cp) {
      l = cl;
      d = cd;
    } else {
      best_match(c, p, &l, &d);
    }
    if (l >= c->m && parse == 1 && p + 1 < n) {
      best_match(c, p + 1, &cl, &cd);
      cp = p + 1;
      if (cl > l) l = 0; /* deferred (R21) */
    }
    if (ntok % 8 == 0) {
      flag_pos = pos;
      tmp[pos++] = 0;
    }
    if (l >= c->m) {
      tmp[flag_pos] |= (uint8_t)(1u << (ntok % 8));
      tmp[pos++] = (uint8_t)((d - 1) & 0xFF);
      tmp[pos++] = (uint8_t)((d - 1) >> 8);
      tmp[pos++] = (uint8_t)(l - c->m);
      p += l;
    } else {
      tmp[pos++] = x[p];
      p += 1;
    }
    ++ntok;
    if (pos >= n) break; /* already not shorter: raw */
  }
  if (pos >= n) {
    memcpy(out, x, n);
    return n;
  }
  memcpy(out, tmp, pos);
  return pos;
}

typedef struct {
  const uint8_t* in;
  size_t n_bytes;
  const lzr_fast_params* prm;
  uint8_t* slots;
  uint32_t* sizes;
  size_t N;
  atomic_size_t next;
} job;

static void* worker(void* arg) {
  job* J = (job*)arg;
  const uint32_t C = J->prm->chunk_size;
  chunk_ctx c;
  c.head = (uint32_t*)calloc(HSIZE, sizeof(uint32_t));
  c.epoch = 0;
  c.prev = (int32_t*)malloc(C * sizeof(int32_t));
  c.run_s = (uint32_t*)malloc(C * sizeof(uint32_t));
  c.run_e = (uint32_t*)malloc(C * sizeof(uint32_t));
  c.run_next = (int32_t*)malloc(C * sizeof(int32_t));
  c.run_of = (int32_t*)malloc(C * sizeof(int32_t));
  uint8_t* buf = (uint8_t*)malloc(C + 16); /* chunk + 8 zero bytes for 8-byte loads */
  uint8_t* tmp = (uint8_t*)malloc(C + C / 8 + 16);
  c.W = J->prm->window;
  c.m = J->prm->min_match;
  c.M = J->prm->max_match;
  c.k = c.m < 4 ? c.m : 4;
  for (;;) {
    const size_t i = atomic_fetch_add(&J->next, 1);
    if (i >= J->N) break;
    const size_t lo = i * C;
    const uint32_t n = (uint32_t)((J->n_bytes - lo) < C ? (J->n_bytes - lo) : C);
    memcpy(buf, J->in + lo, n);
    memset(buf + n, 0, 16);
    c.x = buf;
    c.n = n;
    c.P = n >= c.m ? n - c.m + 1 : 0;
    J->sizes[i] = compress_chunk(&c, J->prm->parse, J->slots + lo, tmp);
  }
  free(c.head);
  free(c.prev);
  free(c.run_s);
  free(c.run_e);
  free(c.run_next);
  free(c.run_of);
  free(buf);
  free(tmp);
  return NULL;
}

int lzr_fast_compress(const uint8_t* in, size_t n_bytes, const lzr_fast_params* prm,
                      uint8_t* slots, uint8_t* out, uint32_t* sizes, uint64_t* offsets,
                      uint64_t* total, int n_threads) {
  const int v = lzr_fast_validate(prm);
  if (v) return v;
  const size_t C = prm->chunk_size;
  const size_t N = (n_bytes + C - 1) / C;
  if (n_threads < 1) n_threads = 1;
  if ((size_t)n_threads > N) n_threads = N ? (int)N : 1;
  job J = {in, n_bytes, prm, slots, sizes, N, 0};
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)n_threads);
  for (int t = 1; t < n_threads; ++t) pthread_create(&th[t], NULL, worker, &J);
  worker(&J);
  for (int t = 1; t < n_threads; ++t) pthread_join(th[t], NULL);
  free(th);
  uint64_t acc = 0;
  for (size_t i = 0; i < N; ++i) {
    offsets[i] = acc;
    acc += sizes[i];
  }
  if (total) *total = acc;
  if (out) /* compaction in chunk order (R11) */
    for (size_t i = 0; i < N; ++i) memmove(out + offsets[i], slots + i * C, sizes[i]);
  return 0;
}
