/*
 * cpuref/lzr_fast.h -- FAST EXACT CPU COMPRESSOR (TEST INFRASTRUCTURE AND CPU
 * BASELINE ONLY).  See lzr_fast.c.  Only tests/, bench.py
 * and tools/ may load it; the product path never does.  It shares no code or
 * header with the CUDA path (include/lzr.h) or with oracle/.
 */
#ifndef LZR_FAST_H
#define LZR_FAST_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct lzr_fast_params {
  uint32_t chunk_size; /* C: 16..65536, multiple of 16                        */
  uint32_t window;     /* W: 1..C                                             */
  uint32_t min_match;  /* m: 3..255                                           */
  uint32_t max_match;  /* M: m..m+255                                         */
  uint32_t tie_break;  /* 0 = longest, then nearest                           */
  uint32_t parse;      /* 0 = greedy (R8), 1 = one-step lazy (R21)            */
} lzr_fast_params;

/* 0, -1 (invalid parameter) or -2 (unsupported tie_break / parse) */
int lzr_fast_validate(const lzr_fast_params* p);

/* Whole stream, thread-per-chunk.  slots: n_bytes of scratch (chunk i's
 * stream at slots + i*C; may equal out: compaction is in place and in order).
 * out: >= n_bytes (may be NULL: sizes/offsets only).  sizes[N], offsets[N]
 * (exclusive prefix sum), *total (may be NULL).  Returns 0 or the validate
 * error. */
int lzr_fast_compress(const uint8_t* in, size_t n_bytes, const lzr_fast_params* prm,
                      uint8_t* slots, uint8_t* out, uint32_t* sizes, uint64_t* offsets,
                      uint64_t* total, int n_threads);

#ifdef __cplusplus
}
#endif
#endif
