/*
 * oracle/lzr_ref.c -- CPU ORACLE (TEST INFRASTRUCTURE ONLY; see lzr_ref.h).
 *
 * Plain serial greedy LZ77 over independent fixed-size chunks, exhaustive
 * longest-match search, flag-byte LZSS encoding, raw fallback.  Written to be
 * checked against the paper and DESIGN.md's readings by eye: no hashing, no
 * candidate filtering, no blocking, no reordering.  Only tests/,
 * __graft_entry__.smoke() and bench.py's CPU baseline legs may use it.
 *
 * Citations:  P:<line> = /root/reference/PAPER.md line (one line = one PDF page).
 * Readings R1..R14 = DESIGN.md §"Readings of the paper" (= SURVEY.md §8(c)).
 */
#include "lzr_ref.h"

#include <pthread.h>
#include <stdlib.h>
#include <string.h>

/* R-params (R1, R3, R4, R7): C multiple of 16 in [16, 65536];
 * 1 <= W <= C; 3 <= m <= 255; m <= M <= m + 255 (8-bit length field);
 * tie_break must be 0 ("longest, then nearest"); parse 0 (greedy, R8) or 1
 * (one-step lazy, R21). */
int lzr_ref_validate(const lzr_ref_params* p) {
  if (!p) return LZR_REF_ERR_INVALID_ARG;
  if (p->chunk_size < 16 || p->chunk_size > 65536 || (p->chunk_size % 16) != 0)
    return LZR_REF_ERR_INVALID_ARG;
  if (p->window < 1 || p->window > p->chunk_size) return LZR_REF_ERR_INVALID_ARG;
  if (p->min_match < 3 || p->min_match > 255) return LZR_REF_ERR_INVALID_ARG;
  if (p->max_match < p->min_match || p->max_match > p->min_match + 255)
    return LZR_REF_ERR_INVALID_ARG;
  if (p->tie_break != 0) return LZR_REF_ERR_UNSUPPORTED;
  if (p->parse > 1) return LZR_REF_ERR_UNSUPPORTED;
  return LZR_REF_OK;
}

/* P:12 §2 "Chunking is the process of breaking a data stream into chunks";
 * the last chunk may be short (R10). */
size_t lzr_ref_num_chunks(size_t n_bytes, const lzr_ref_params* p) {
  return (n_bytes + p->chunk_size - 1) / p->chunk_size;
}

/* P:12 §2: a repeated sequence in the look-ahead buffer (x[p..]) is replaced
 * by a pointer into the history buffer (the W bytes before p in the same
 * chunk, R2).  For d = 1 .. min(W, p), ascending:
 *     l(d) = number of leading k < cap with x[p+k] == x[p-d+k],
 *     cap  = min(M, n - p)                    (R3, R6: cap before tie-break)
 * Overlap (d < l) compares against the original bytes, which is exactly what
 * byte-serial copying reproduces on decode (R5).  Keep the first d with the
 * largest l (strict '>' => nearest wins ties, R7); stop once l == cap since
 * nothing can beat the cap. */
void lzr_ref_best_match(const uint8_t* x, size_t n, size_t p, const lzr_ref_params* prm,
                        uint32_t* len, uint32_t* dist) {
  size_t cap = n - p;
  if (cap > prm->max_match) cap = prm->max_match;
  size_t dmax = p < prm->window ? p : prm->window;
  size_t best = 0, bd = 0;
  for (size_t d = 1; d <= dmax; ++d) {
    size_t l = 0;
    while (l < cap && x[p + l] == x[p - d + l]) ++l;
    if (l > best) {
      best = l;
      bd = d;
      if (best == cap) break;
    }
  }
  *len = (uint32_t)best;
  *dist = (uint32_t)bd;
}

/* Greedy parse (R8; §3.2(2) post-processing, whose rule the paper does
 * not give): p = 0; while p < n: take the best match if its length >= m,
 * else a literal.
 * One-step lazy parse (R21, parse = 1; SURVEY.md §8(f) N4 "lazy matching"):
 * the same, except that a match at p is deferred -- x[p] is emitted as a
 * literal and the walk moves to p + 1 -- when the best match at p + 1 is
 * strictly longer than the one at p.  The decision at p depends on p alone. */
size_t lzr_ref_parse_chunk(const uint8_t* x, size_t n, const lzr_ref_params* prm,
                           uint32_t* lens, uint32_t* dists) {
  size_t p = 0, t = 0;
  while (p < n) {
    uint32_t l, d;
    lzr_ref_best_match(x, n, p, prm, &l, &d);
    int take = l >= prm->min_match;
    if (take && prm->parse == 1 && p + 1 < n) {
      uint32_t l1, d1;
      lzr_ref_best_match(x, n, p + 1, prm, &l1, &d1);
      if (l1 > l) take = 0; /* a longer match starts at p + 1: literal now */
    }
    if (take) {
      lens[t] = l;
      dists[t] = d;
      p += l;
    } else {
      lens[t] = 1;
      dists[t] = 0;
      p += 1;
    }
    ++t;
  }
  return t;
}

/* Flag-byte LZSS (R1): a group is one flag byte followed by up to 8 tokens;
 * flag bit i (LSB first) = 1 means token i of the group is a match.
 * Literal = 1 byte.  Match = 3 bytes: (d-1) as uint16 little-endian, then
 * (l-m) as uint8.  Unused flag bits of the last group are 0; no end marker. */
typedef struct {
  uint8_t* buf;
  size_t pos;
  size_t flag_pos;
  size_t ntok;
} ref_encoder;

static void enc_open_group_if_needed(ref_encoder* e) {
  if (e->ntok % 8 == 0) {
    e->flag_pos = e->pos;
    e->buf[e->pos++] = 0;
  }
}

static void enc_literal(ref_encoder* e, uint8_t b) {
  enc_open_group_if_needed(e);
  e->buf[e->pos++] = b;
  e->ntok++;
}

static void enc_match(ref_encoder* e, uint32_t d, uint32_t l, uint32_t m) {
  enc_open_group_if_needed(e);
  e->buf[e->flag_pos] |= (uint8_t)(1u << (e->ntok % 8));
  e->buf[e->pos++] = (uint8_t)((d - 1) & 0xFF);
  e->buf[e->pos++] = (uint8_t)((d - 1) >> 8);
  e->buf[e->pos++] = (uint8_t)(l - m);
  e->ntok++;
}

/* One chunk: parse, encode, then raw fallback (R9): if S >= n the chunk is
 * stored verbatim and S := n.  (S == n is therefore the "raw" sentinel.) */
size_t lzr_ref_compress_chunk(const uint8_t* x, size_t n, const lzr_ref_params* prm,
                              uint8_t* out) {
  if (n == 0) return 0;
  uint32_t* lens = (uint32_t*)malloc(n * sizeof(uint32_t));
  uint32_t* dists = (uint32_t*)malloc(n * sizeof(uint32_t));
  /* worst case: n literals + ceil(n/8) flag bytes */
  uint8_t* tmp = (uint8_t*)malloc(n + n / 8 + 16);
  size_t T = lzr_ref_parse_chunk(x, n, prm, lens, dists);
  ref_encoder e = {tmp, 0, 0, 0};
  size_t p = 0;
  for (size_t t = 0; t < T; ++t) {
    if (dists[t] == 0) {
      enc_literal(&e, x[p]);
    } else {
      enc_match(&e, dists[t], lens[t], prm->min_match);
    }
    p += lens[t];
  }
  size_t S = e.pos;
  if (S >= n) {
    memcpy(out, x, n);
    S = n;
  } else {
    memcpy(out, tmp, S);
  }
  free(tmp);
  free(dists);
  free(lens);
  return S;
}

/* Decoder (inverse of R1): S == n -> verbatim copy.  Otherwise read groups
 * until n bytes are produced; a match copies byte by byte from op - d, which
 * reproduces overlapping matches (R5).  Corrupt if: S > n; a token runs past S;
 * d > bytes produced so far; a match overruns n; the stream has bytes left
 * after n bytes are produced; or unused flag bits of the last group are set. */
int lzr_ref_decompress_chunk(const uint8_t* s, size_t S, size_t n, const lzr_ref_params* prm,
                             uint8_t* out) {
  if (S == n) {
    memcpy(out, s, n);
    return LZR_REF_OK;
  }
  if (S > n) return LZR_REF_ERR_CORRUPT;
  size_t ip = 0, op = 0;
  while (op < n) {
    if (ip >= S) return LZR_REF_ERR_CORRUPT;
    uint32_t f = s[ip++];
    for (uint32_t bit = 0; bit < 8; ++bit) {
      if (op == n) {
        if ((f >> bit) != 0) return LZR_REF_ERR_CORRUPT;
        break;
      }
      if (f & (1u << bit)) {
        if (ip + 3 > S) return LZR_REF_ERR_CORRUPT;
        size_t d = (size_t)s[ip] + ((size_t)s[ip + 1] << 8) + 1;
        size_t l = (size_t)s[ip + 2] + prm->min_match;
        ip += 3;
        if (d > op) return LZR_REF_ERR_CORRUPT;
        if (op + l > n) return LZR_REF_ERR_CORRUPT;
        for (size_t k = 0; k < l; ++k) out[op + k] = out[op - d + k];
        op += l;
      } else {
        if (ip >= S) return LZR_REF_ERR_CORRUPT;
        out[op++] = s[ip++];
      }
    }
  }
  if (ip != S) return LZR_REF_ERR_CORRUPT;
  return LZR_REF_OK;
}

/* ---- thread-per-chunk drivers (§3.2(1)) ---------------------------- */

typedef struct {
  const uint8_t* in;
  size_t n_bytes;
  const lzr_ref_params* prm;
  const uint64_t* idx; /* NULL: chunk j = j */
  size_t n_jobs;
  uint8_t* slots; /* n_jobs * chunk_size */
  uint32_t* sizes;
  size_t next;
  pthread_mutex_t mu;
} ref_job;

static void* ref_worker(void* arg) {
  ref_job* j = (ref_job*)arg;
  const size_t C = j->prm->chunk_size;
  for (;;) {
    pthread_mutex_lock(&j->mu);
    size_t k = j->next++;
    pthread_mutex_unlock(&j->mu);
    if (k >= j->n_jobs) break;
    size_t c = j->idx ? (size_t)j->idx[k] : k;
    size_t lo = c * C;
    size_t ni = j->n_bytes - lo < C ? j->n_bytes - lo : C;
    j->sizes[k] = (uint32_t)lzr_ref_compress_chunk(j->in + lo, ni, j->prm, j->slots + k * C);
  }
  return NULL;
}

static void ref_run(ref_job* job, int n_threads) {
  if (n_threads < 1) n_threads = 1;
  if ((size_t)n_threads > job->n_jobs) n_threads = job->n_jobs ? (int)job->n_jobs : 1;
  pthread_mutex_init(&job->mu, NULL);
  job->next = 0;
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)n_threads);
  for (int t = 0; t < n_threads; ++t) pthread_create(&th[t], NULL, ref_worker, job);
  for (int t = 0; t < n_threads; ++t) pthread_join(th[t], NULL);
  free(th);
  pthread_mutex_destroy(&job->mu);
}

/* R11: output compacted in chunk order; offsets = exclusive prefix sum of sizes. */
int lzr_ref_compress(const uint8_t* in, size_t n_bytes, const lzr_ref_params* prm,
                     uint8_t* out, size_t out_capacity, uint32_t* sizes, uint64_t* offsets,
                     uint64_t* total, int n_threads) {
  int st = lzr_ref_validate(prm);
  if (st) return st;
  size_t N = lzr_ref_num_chunks(n_bytes, prm);
  if (out_capacity < n_bytes) return LZR_REF_ERR_CAPACITY;
  if (N == 0) {
    if (total) *total = 0;
    return LZR_REF_OK;
  }
  ref_job job;
  memset(&job, 0, sizeof job);
  job.in = in;
  job.n_bytes = n_bytes;
  job.prm = prm;
  job.idx = NULL;
  job.n_jobs = N;
  job.slots = (uint8_t*)malloc(N * (size_t)prm->chunk_size);
  job.sizes = sizes;
  ref_run(&job, n_threads);
  uint64_t acc = 0;
  for (size_t i = 0; i < N; ++i) {
    offsets[i] = acc;
    memcpy(out + acc, job.slots + i * (size_t)prm->chunk_size, sizes[i]);
    acc += sizes[i];
  }
  if (total) *total = acc;
  free(job.slots);
  return LZR_REF_OK;
}

int lzr_ref_compress_sampled(const uint8_t* in, size_t n_bytes, const lzr_ref_params* prm,
                             const uint64_t* idx, size_t n_idx, uint8_t* out, uint32_t* sizes,
                             int n_threads) {
  int st = lzr_ref_validate(prm);
  if (st) return st;
  size_t N = lzr_ref_num_chunks(n_bytes, prm);
  for (size_t k = 0; k < n_idx; ++k)
    if (idx[k] >= N) return LZR_REF_ERR_INVALID_ARG;
  ref_job job;
  memset(&job, 0, sizeof job);
  job.in = in;
  job.n_bytes = n_bytes;
  job.prm = prm;
  job.idx = idx;
  job.n_jobs = n_idx;
  job.slots = out;
  job.sizes = sizes;
  ref_run(&job, n_threads);
  return LZR_REF_OK;
}

int lzr_ref_decompress(const uint8_t* comp, const uint32_t* sizes, const uint64_t* offsets,
                       size_t n_bytes, const lzr_ref_params* prm, uint8_t* out,
                       int32_t* first_bad) {
  int st = lzr_ref_validate(prm);
  if (st) return st;
  size_t N = lzr_ref_num_chunks(n_bytes, prm);
  const size_t C = prm->chunk_size;
  if (first_bad) *first_bad = 0;
  for (size_t i = 0; i < N; ++i) {
    size_t lo = i * C;
    size_t ni = n_bytes - lo < C ? n_bytes - lo : C;
    if (lzr_ref_decompress_chunk(comp + offsets[i], sizes[i], ni, prm, out + lo) != 0) {
      if (first_bad) *first_bad = (int32_t)(i + 1);
      return LZR_REF_ERR_CORRUPT;
    }
  }
  return LZR_REF_OK;
}
