/*
 * oracle/dedup_ref.c -- CPU oracle of the dedup fingerprint step.
 * TEST INFRASTRUCTURE ONLY: used by tests/, __graft_entry__.smoke() and
 * bench.py's CPU-baseline legs; the product path never links it, and it shares
 * no code with the CUDA path.
 *
 * What it computes:
 *   fp[i] = SHA-1 of chunk i's bytes, chunk i = [iC, min(n, (i+1)C)).
 *   PAPER.md P:12 §2 "Hashing is the process of calculating the hash value of
 *   each chunk. The hash value is used as an identifier for the chunk";
 *   P:14 §3.1(1) "the hash size (SHA1, 20 bytes)".
 * SHA-1 is written out plainly from its standard definition (FIPS 180-4 §5.1.1
 * padding, §6.1.2 computation, §4.1.1 functions, §4.2.1 constants); pins:
 * tests/test_dedup_oracle.py (FIPS example digests, hashlib on random inputs,
 * every length 0..300 around the padding boundaries).
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static uint32_t rotl(uint32_t x, int s) { return (x << s) | (x >> (32 - s)); }

/* one 512-bit block (FIPS 180-4 §6.1.2 steps 1-4) */
static void sha1_block(uint32_t H[5], const uint8_t* blk) {
  uint32_t W[80];
  for (int t = 0; t < 16; ++t)
    W[t] = ((uint32_t)blk[4 * t] << 24) | ((uint32_t)blk[4 * t + 1] << 16) |
           ((uint32_t)blk[4 * t + 2] << 8) | (uint32_t)blk[4 * t + 3];
  for (int t = 16; t < 80; ++t) W[t] = rotl(W[t - 3] ^ W[t - 8] ^ W[t - 14] ^ W[t - 16], 1);
  uint32_t a = H[0], b = H[1], c = H[2], d = H[3], e = H[4];
  for (int t = 0; t < 80; ++t) {
    uint32_t f, K;
    if (t < 20) {
      f = (b & c) ^ (~b & d);  /* Ch */
      K = 0x5a827999u;
    } else if (t < 40) {
      f = b ^ c ^ d;           /* Parity */
      K = 0x6ed9eba1u;
    } else if (t < 60) {
      f = (b & c) ^ (b & d) ^ (c & d);  /* Maj */
      K = 0x8f1bbcdcu;
    } else {
      f = b ^ c ^ d;
      K = 0xca62c1d6u;
    }
    uint32_t T = rotl(a, 5) + f + e + K + W[t];
    e = d;
    d = c;
    c = rotl(b, 30);
    b = a;
    a = T;
  }
  H[0] += a;
  H[1] += b;
  H[2] += c;
  H[3] += d;
  H[4] += e;
}

/* SHA-1 of msg[0..len) -> 20-byte big-endian digest (FIPS 180-4 §5.1.1 padding:
   0x80, zeros to 56 mod 64, 64-bit big-endian bit length) */
void dedup_ref_sha1(const uint8_t* msg, size_t len, uint8_t out[20]) {
  uint32_t H[5] = {0x67452301u, 0xefcdab89u, 0x98badcfeu, 0x10325476u, 0xc3d2e1f0u};
  size_t i = 0;
  for (; i + 64 <= len; i += 64) sha1_block(H, msg + i);
  uint8_t tail[128];
  size_t r = len - i;
  memset(tail, 0, sizeof(tail));
  memcpy(tail, msg + i, r);
  tail[r] = 0x80;
  size_t tl = (r + 1 + 8 <= 64) ? 64 : 128;
  uint64_t bits = (uint64_t)len * 8u;
  for (int k = 0; k < 8; ++k) tail[tl - 1 - k] = (uint8_t)(bits >> (8 * k));
  sha1_block(H, tail);
  if (tl == 128) sha1_block(H, tail + 64);
  for (int k = 0; k < 5; ++k) {
    out[4 * k] = (uint8_t)(H[k] >> 24);
    out[4 * k + 1] = (uint8_t)(H[k] >> 16);
    out[4 * k + 2] = (uint8_t)(H[k] >> 8);
    out[4 * k + 3] = (uint8_t)H[k];
  }
}

typedef struct {
  const uint8_t* in;
  size_t n, C, N;
  uint8_t* fp;
  int tid, nthr;
} job_t;

static void* worker(void* arg) {
  job_t* j = (job_t*)arg;
  for (size_t i = (size_t)j->tid; i < j->N; i += (size_t)j->nthr) {
    size_t lo = i * j->C;
    size_t len = j->n - lo < j->C ? j->n - lo : j->C;
    dedup_ref_sha1(j->in + lo, len, j->fp + 20 * i);
  }
  return NULL;
}

/* fp[i] (20 bytes each) for every chunk of in[0..n); thread-per-chunk
   (chunks are independent: §3.1 "no data dependency between chunks when the
   hash value of the chunk is calculated") */
int dedup_ref_fingerprints(const uint8_t* in, size_t n, size_t C, uint8_t* fp, int n_threads) {
  if (C == 0) return -1;
  size_t N = (n + C - 1) / C;
  if (n_threads < 1) n_threads = 1;
  if (n_threads > 256) n_threads = 256;
  pthread_t th[256];
  job_t jobs[256];
  for (int t = 0; t < n_threads; ++t) {
    jobs[t] = (job_t){in, n, C, N, fp, t, n_threads};
    if (pthread_create(&th[t], NULL, worker, &jobs[t])) return -4;
  }
  for (int t = 0; t < n_threads; ++t) pthread_join(th[t], NULL);
  return 0;
}
