/* synth/synth_host.c -- host side of the seeded generator (see synth_core.h). */
#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

#include "synth_core.h"

/* Vocabulary and Zipf(1.1) CDF derived from the seed.  Built once on the host;
 * the device generator receives a copy of the same bytes, so both sides use
 * identical tables. */
void syn_build_tables(uint64_t seed, syn_tables* t) {
  double w[SYN_VOCAB], sum = 0.0;
  for (int r = 0; r < SYN_VOCAB; ++r) {
    w[r] = 1.0 / pow((double)(r + 1), 1.1);
    sum += w[r];
  }
  double acc = 0.0;
  uint32_t prev = 0;
  for (int r = 0; r < SYN_VOCAB; ++r) {
    acc += w[r];
    double c = acc / sum * 4294967296.0;
    uint32_t v = c >= 4294967295.0 ? 0xFFFFFFFFu : (uint32_t)c;
    if (r > 0 && v <= prev) v = prev + 1;
    t->cdf[r] = v;
    prev = v;
  }
  t->cdf[SYN_VOCAB - 1] = 0xFFFFFFFFu;
  for (int k = 0; k < SYN_VOCAB; ++k) {
    syn_rng g;
    g.s = syn_mix(seed ^ 0x70CAB0000ull ^ ((uint64_t)k * SYN_GOLDEN));
    uint64_t v = syn_next(&g);
    uint32_t L = 3u + (uint32_t)(v % 7u);
    t->wlen[k] = (uint8_t)L;
    memset(t->word[k], 0, sizeof t->word[k]);
    for (uint32_t j = 0; j < L; ++j) {
      v = syn_next(&g);
      t->word[k][j] = (uint8_t)('a' + (v % 26u));
    }
  }
}

size_t syn_tables_bytes(void) { return sizeof(syn_tables); }

typedef struct {
  uint8_t* out;
  size_t n;
  uint32_t C;
  int cls;
  uint64_t seed, first;
  const syn_tables* t;
  size_t N, next;
  pthread_mutex_t mu;
} syn_job;

static void* syn_worker(void* a) {
  syn_job* j = (syn_job*)a;
  for (;;) {
    pthread_mutex_lock(&j->mu);
    size_t lo = j->next;
    j->next += 64;
    pthread_mutex_unlock(&j->mu);
    if (lo >= j->N) break;
    size_t hi = lo + 64 < j->N ? lo + 64 : j->N;
    for (size_t i = lo; i < hi; ++i) {
      size_t b = i * j->C;
      uint32_t ni = (uint32_t)(j->n - b < j->C ? j->n - b : j->C);
      syn_fill_chunk(j->out + b, ni, j->cls, j->seed, j->first + i, j->t);
    }
  }
  return NULL;
}

/* Fill out[0..n) with chunks first_chunk, first_chunk+1, ... of class cls. */
int syn_fill(uint8_t* out, size_t n, uint32_t chunk_size, int cls, uint64_t seed,
             uint64_t first_chunk, const syn_tables* t, int n_threads) {
  if (chunk_size == 0 || cls < 0 || (cls & ~SYN_DEDUP) >= SYN_NCLASS) return -1;
  syn_job j;
  memset(&j, 0, sizeof j);
  j.out = out; j.n = n; j.C = chunk_size; j.cls = cls; j.seed = seed; j.first = first_chunk;
  j.t = t; j.N = (n + chunk_size - 1) / chunk_size; j.next = 0;
  pthread_mutex_init(&j.mu, NULL);
  if (n_threads < 1) n_threads = 1;
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)n_threads);
  for (int k = 0; k < n_threads; ++k) pthread_create(&th[k], NULL, syn_worker, &j);
  for (int k = 0; k < n_threads; ++k) pthread_join(th[k], NULL);
  free(th);
  pthread_mutex_destroy(&j.mu);
  return 0;
}

int syn_chunk_class_of(int cls, uint64_t seed, uint64_t chunk) {
  return syn_chunk_class(cls, seed, chunk);
}

uint64_t syn_dedup_source_of(uint64_t seed, uint64_t chunk) { return syn_dedup_source(seed, chunk); }
