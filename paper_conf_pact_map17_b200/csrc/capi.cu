// capi.cu -- the extern "C" boundary of liblzr.so (include/lzr.h): parameter
// validation, workspace sizing, launch sequencing on the caller's stream, and
// the host-buffer end-to-end pipeline.  No device memory is allocated here.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>

#include "lzr_internal.cuh"

namespace lzr {

namespace {

struct DevInfo {
  int sm_count = 0;
  int smem_optin = 0;
};

thread_local int t_launches = 0;
std::mutex g_mu;
DevInfo g_dev[64];

cudaError_t dev_info(DevInfo* out) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lk(g_mu);
  if (g_dev[dev].sm_count == 0) {
    int sms = 0, smem = 0;
    e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) return e;
    e = cudaDeviceGetAttribute(&smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    if (e != cudaSuccess) return e;
    g_dev[dev].sm_count = sms;
    g_dev[dev].smem_optin = smem;
  }
  *out = g_dev[dev];
  return cudaSuccess;
}

bool aligned(const void* p, size_t a) { return ((uintptr_t)p % a) == 0; }

// Warps cooperating on one chunk (K): 4 up to 4 KiB chunks, 8 up to 8 KiB
// (fewer chunks fit one SM's shared memory, so each gets more warps), 16 up to
// 16 KiB with the walk bitmaps in the L2 scratch and <= 56 registers (two
// chunks of 16 warps per SM), 32 above (one chunk of 32 warps per SM, <= 64
// registers).  1 x B200, 1 GiB mix, GB/s: 16 KiB 25.9 (K = 8) -> 33.7 (16) /
// 25.6 (32); 32 KiB 12.0 (8) -> 17.8 (16) -> 24.0 (32); 64 KiB 11.8 (16) ->
// 16.7 (32); at 8 KiB 16 warps lose to four groups of 8: 34.1 vs 44.0.
// LZR_ENCODE_WARPS=1,2,3,4,8 overrides (tuning).
// chunks above this size get 16 warps (walk bitmaps in the L2 scratch)
#ifndef LZR_K16_MIN
#define LZR_K16_MIN 8192
#endif
#ifndef LZR_K32_MIN
#define LZR_K32_MIN 16384
#endif
uint32_t enc_warps_per_chunk(uint32_t C) {
  static int env = -1;
  if (env < 0) {
    const char* e = getenv("LZR_ENCODE_WARPS");
    env = (e && ((*e >= '1' && *e <= '4') || *e == '8')) ? (*e - '0') : 0;
  }
  if (C > kBigChunk) return LZR_BIG_WARPS;  // the big-chunk layout (lzr_internal.cuh)
  if (env > 0) return (uint32_t)env;
  return C > LZR_K32_MIN ? 32u : (C > LZR_K16_MIN ? 16u : (C > 4096 ? 8u : (C >= 1024 ? 4u : 1u)));
}

// big chunks: two scatter splits of 4096 buckets each (1 x B200, 1 GiB, 64 KiB
// chunks, mix/text/zero-runs GB/s: 1 split of 8192 buckets 10.5/5.2/22.0,
// 2 splits 11.8/5.6/32.1, 4 splits 10.5/4.9/35.7)
#ifndef LZR_BIG_SPLITS
#define LZR_BIG_SPLITS 2u
#endif
// warps that share the index scatter (each a contiguous position range with
// its own cursor array; the hash table shrinks by the same factor)
uint32_t enc_scatter_splits(uint32_t K, uint32_t C) {
  static int env = -1;
  if (env < 0) {
    const char* e = getenv("LZR_ENCODE_SPLITS");
    env = (e && (*e == '1' || *e == '2' || *e == '4' || *e == '8')) ? (*e - '0') : 0;
  }
  // default (config-3 sweep, 1 x B200): 1 split at K = 4 (C = 4 KiB: the full
  // C-bucket table matters more than the serial scatter), 4 at K = 8
  if (K > 8) {  // big chunks: NS splits share the slot region's 8192 counters
    if (C > kBigChunk) return env == 2 || env == 4 ? (uint32_t)env : LZR_BIG_SPLITS;
    return 4u;
  }
  const uint32_t ns = env > 0 ? (uint32_t)env : (K >= 8 ? 4u : 1u);
  return K < 4 ? 1u : (ns < K ? ns : K);  // (kernels are instantiated for these)
}

}  // namespace

WsLayout ws_layout(size_t n_bytes, const lzr_params* p) {
  WsLayout w;
  const size_t C = p->chunk_size;
  const size_t N = (n_bytes + C - 1) / C;
  DevInfo di;
  const size_t sms = dev_info(&di) == cudaSuccess ? (size_t)di.sm_count : 1024;
  // resident chunk groups: grid (<= SMs x CTAs per SM) x groups per CTA; both
  // bounded by one SM's shared memory (228 KB) over a group's footprint, and
  // by 16 per SM; the launch uses at most ceil(N / groups) CTAs, i.e. at most
  // N + 15 groups
  const uint32_t K = enc_warps_per_chunk((uint32_t)C);
  const EncLayout L = enc_layout((uint32_t)C, K, enc_scatter_splits(K, (uint32_t)C));
  size_t per_sm = kSmemPerSm / L.per_group;
  if (per_sm > kMaxGroupsPerSm) per_sm = kMaxGroupsPerSm;
  if (per_sm < 1) per_sm = 1;
  size_t groups = sms * per_sm;
  if (groups > N + kMaxGroupsPerSm) groups = N + kMaxGroupsPerSm;
  w.ctrl_off = 0;
  w.slots_off = 256;
  w.scratch_off = w.slots_off + align_up_z(N * C, 256);
  w.scan_off = w.scratch_off + align_up_z(groups * enc_scratch_per_group(L, (uint32_t)C), 256);
  w.total = w.scan_off + scan_ws_bytes(N);
  return w;
}

}  // namespace lzr

using namespace lzr;

extern "C" {

int lzr_validate_params(const lzr_params* p) {
  if (!p) return LZR_ERR_INVALID_ARG;
  if (p->chunk_size < 16 || p->chunk_size > 65536 || p->chunk_size % 16) return LZR_ERR_INVALID_ARG;
  if (p->window < 1 || p->window > p->chunk_size) return LZR_ERR_INVALID_ARG;
  if (p->min_match < 3 || p->min_match > 255) return LZR_ERR_INVALID_ARG;
  if (p->max_match < p->min_match || p->max_match > p->min_match + 255) return LZR_ERR_INVALID_ARG;
  if (p->tie_break != LZR_TIE_LONGEST_THEN_NEAREST) return LZR_ERR_UNSUPPORTED;
  if (p->parse != LZR_PARSE_GREEDY && p->parse != LZR_PARSE_LAZY) return LZR_ERR_UNSUPPORTED;
  return LZR_OK;
}

size_t lzr_num_chunks(size_t n_bytes, const lzr_params* p) {
  if (lzr_validate_params(p) != LZR_OK) return 0;
  return (n_bytes + p->chunk_size - 1) / p->chunk_size;
}

size_t lzr_compress_bound(size_t n_bytes, const lzr_params* p) {
  if (lzr_validate_params(p) != LZR_OK) return 0;
  return n_bytes;
}

size_t lzr_compress_workspace_bytes(size_t n_bytes, const lzr_params* p) {
  if (lzr_validate_params(p) != LZR_OK) return 0;
  return ws_layout(n_bytes, p).total;
}

size_t lzr_scan_workspace_bytes(size_t n) { return scan_ws_bytes(n); }

int lzr_last_launch_count(void) { return t_launches; }

const char* lzr_status_str(int s) {
  switch (s) {
    case LZR_OK: return "LZR_OK";
    case LZR_ERR_INVALID_ARG: return "LZR_ERR_INVALID_ARG";
    case LZR_ERR_UNSUPPORTED: return "LZR_ERR_UNSUPPORTED";
    case LZR_ERR_CAPACITY: return "LZR_ERR_CAPACITY";
    case LZR_ERR_CUDA: return "LZR_ERR_CUDA";
    case LZR_ERR_CORRUPT: return "LZR_ERR_CORRUPT";
    default: return "LZR_ERR_UNKNOWN";
  }
}

int lzr_compress_encode(const void* d_in, size_t n_bytes, const lzr_params* p, uint32_t* d_sizes,
                        void* d_workspace, size_t workspace_bytes, lzr_stream_t stream) {
  t_launches = 0;
  int st = lzr_validate_params(p);
  if (st) return st;
  if (n_bytes == 0) return LZR_OK;
  if (!d_in || !d_sizes || !d_workspace) return LZR_ERR_INVALID_ARG;
  if (!aligned(d_in, 16) || !aligned(d_sizes, 4) || !aligned(d_workspace, 256))
    return LZR_ERR_INVALID_ARG;
  const WsLayout w = ws_layout(n_bytes, p);
  if (workspace_bytes < w.total) return LZR_ERR_CAPACITY;
  const size_t N = (n_bytes + p->chunk_size - 1) / p->chunk_size;
  if (N > 0xFFFFFFFFull) return LZR_ERR_UNSUPPORTED;
  DevInfo di;
  if (dev_info(&di) != cudaSuccess) return LZR_ERR_CUDA;
  EncArgs a;
  a.in = (const uint8_t*)d_in;
  a.n_bytes = n_bytes;
  a.N = (uint32_t)N;
  a.C = p->chunk_size;
  a.W = p->window;
  a.m = p->min_match;
  a.M = p->max_match;
  a.lazy = p->parse == LZR_PARSE_LAZY;
  a.kbytes = p->min_match < 4 ? p->min_match : 4;
  a.kmask = a.kbytes == 4 ? 0xFFFFFFFFu : ((1u << (8 * a.kbytes)) - 1u);
  const uint32_t K = enc_warps_per_chunk(p->chunk_size);
  a.L = enc_layout(p->chunk_size, K, enc_scatter_splits(K, p->chunk_size));
  // one chunk's index must fit one CTA's shared memory (C <= 32 KiB: 15-bit
  // positions + bucket-start marks; above: the big-chunk layout)
  if ((int)a.L.per_group > di.smem_optin) return LZR_ERR_UNSUPPORTED;
  uint8_t* ws = (uint8_t*)d_workspace;
  a.slots = ws + w.slots_off;
  a.scratch = ws + w.scratch_off;
  a.sizes = d_sizes;
  a.counter = (uint32_t*)(ws + w.ctrl_off);
  cudaStream_t s = (cudaStream_t)stream;
  if (cudaMemsetAsync(ws + w.ctrl_off, 0, 256, s) != cudaSuccess) return LZR_ERR_CUDA;
  if (launch_encode(a, di.sm_count, di.smem_optin, s, &t_launches) != cudaSuccess) return LZR_ERR_CUDA;
  return LZR_OK;
}

int lzr_compress_compact(const void* d_in, size_t n_bytes, const lzr_params* p, void* d_out,
                         size_t out_capacity, const uint32_t* d_sizes, uint64_t* d_offsets,
                         uint64_t* d_total, void* d_workspace, size_t workspace_bytes,
                         lzr_stream_t stream) {
  t_launches = 0;
  int st = lzr_validate_params(p);
  if (st) return st;
  cudaStream_t s = (cudaStream_t)stream;
  if (n_bytes == 0) {
    if (d_total && cudaMemsetAsync(d_total, 0, 8, s) != cudaSuccess) return LZR_ERR_CUDA;
    return LZR_OK;
  }
  if (!d_in || !d_out || !d_sizes || !d_offsets || !d_workspace) return LZR_ERR_INVALID_ARG;
  if (!aligned(d_in, 16) || !aligned(d_sizes, 4) || !aligned(d_offsets, 8) ||
      !aligned(d_workspace, 256) || (d_total && !aligned(d_total, 8)))
    return LZR_ERR_INVALID_ARG;
  if (out_capacity < n_bytes) return LZR_ERR_CAPACITY;
  const WsLayout w = ws_layout(n_bytes, p);
  if (workspace_bytes < w.total) return LZR_ERR_CAPACITY;
  DevInfo di;
  if (dev_info(&di) != cudaSuccess) return LZR_ERR_CUDA;
  const size_t N = (n_bytes + p->chunk_size - 1) / p->chunk_size;
  uint8_t* ws = (uint8_t*)d_workspace;
  if (launch_scan(d_sizes, N, 0, nullptr, d_offsets, d_total, ws + w.scan_off, s, &t_launches) !=
      cudaSuccess)
    return LZR_ERR_CUDA;
  if (launch_compact((const uint8_t*)d_in, n_bytes, p->chunk_size, ws + w.slots_off,
                     (size_t)p->chunk_size, d_sizes,
                     d_offsets, (uint8_t*)d_out, di.sm_count, s, &t_launches) != cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

int lzr_compress_chunks(const void* d_in, size_t n_bytes, const lzr_params* p, void* d_out,
                        size_t out_capacity, uint32_t* d_sizes, uint64_t* d_offsets,
                        uint64_t* d_total, void* d_workspace, size_t workspace_bytes,
                        lzr_stream_t stream) {
  int st = lzr_validate_params(p);
  if (st) return st;
  if (n_bytes && out_capacity < n_bytes) return LZR_ERR_CAPACITY;
  if (n_bytes && (!d_out || !d_offsets)) return LZR_ERR_INVALID_ARG;
  st = lzr_compress_encode(d_in, n_bytes, p, d_sizes, d_workspace, workspace_bytes, stream);
  if (st) return st;
  const int l1 = t_launches;
  st = lzr_compress_compact(d_in, n_bytes, p, d_out, out_capacity, d_sizes, d_offsets, d_total,
                            d_workspace, workspace_bytes, stream);
  t_launches += l1;
  return st;
}

int lzr_scan_sizes(const uint32_t* d_sizes, size_t n, uint64_t base, uint64_t* d_offsets,
                   uint64_t* d_total, void* d_workspace, size_t workspace_bytes,
                   lzr_stream_t stream) {
  t_launches = 0;
  cudaStream_t s = (cudaStream_t)stream;
  if (n == 0) {
    if (d_total) {
      // *d_total = base
      if (cudaMemcpyAsync(d_total, &base, 8, cudaMemcpyHostToDevice, s) != cudaSuccess)
        return LZR_ERR_CUDA;
      if (cudaStreamSynchronize(s) != cudaSuccess) return LZR_ERR_CUDA;
    }
    return LZR_OK;
  }
  if (!d_sizes || !d_offsets || !d_workspace) return LZR_ERR_INVALID_ARG;
  if (!aligned(d_sizes, 4) || !aligned(d_offsets, 8) || !aligned(d_workspace, 256) ||
      (d_total && !aligned(d_total, 8)))
    return LZR_ERR_INVALID_ARG;
  if (workspace_bytes < scan_ws_bytes(n)) return LZR_ERR_CAPACITY;
  if (launch_scan(d_sizes, n, base, nullptr, d_offsets, d_total, d_workspace, s, &t_launches) !=
      cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

int lzr_fingerprint_chunks(const void* d_in, size_t n_bytes, uint32_t chunk_size, uint8_t* d_fp,
                           lzr_stream_t stream) {
  t_launches = 0;
  if (n_bytes == 0) return LZR_OK;
  if (!d_in || !d_fp || chunk_size == 0) return LZR_ERR_INVALID_ARG;
  if (launch_sha1((const uint8_t*)d_in, n_bytes, chunk_size, d_fp, (cudaStream_t)stream,
                  &t_launches) != cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

size_t lzr_dedup_table_bytes(uint32_t n_bins, uint32_t bin_slots) {
  return (size_t)n_bins * bin_slots * dedup_entry_bytes();
}

int lzr_dedup_index(const uint8_t* d_fp, size_t n_chunks, uint64_t first_chunk, void* d_table,
                    uint32_t n_bins, uint32_t bin_slots, uint64_t* d_index, uint32_t* d_unique,
                    uint32_t* d_overflow, lzr_stream_t stream) {
  t_launches = 0;
  if (n_chunks == 0) return LZR_OK;
  if (!d_fp || !d_table || !d_index || !d_unique || !d_overflow || n_bins == 0 || bin_slots == 0)
    return LZR_ERR_INVALID_ARG;
  if (!aligned(d_table, 256) || !aligned(d_index, 8) || !aligned(d_unique, 4) ||
      !aligned(d_overflow, 4))
    return LZR_ERR_INVALID_ARG;
  if (launch_index(d_fp, n_chunks, first_chunk, nullptr, d_table, n_bins, bin_slots, d_index,
                   d_unique, d_overflow, (cudaStream_t)stream, &t_launches) != cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

int lzr_dedup_index_gidx(const uint8_t* d_fp, size_t n, const uint64_t* d_gidx, void* d_table,
                         uint32_t n_bins, uint32_t bin_slots, uint64_t* d_index, uint32_t* d_unique,
                         uint32_t* d_overflow, lzr_stream_t stream) {
  t_launches = 0;
  if (n == 0) return LZR_OK;
  if (!d_fp || !d_gidx || !d_table || !d_index || !d_unique || !d_overflow || n_bins == 0 ||
      bin_slots == 0)
    return LZR_ERR_INVALID_ARG;
  if (!aligned(d_table, 256) || !aligned(d_gidx, 8) || !aligned(d_index, 8) || !aligned(d_unique, 4) ||
      !aligned(d_overflow, 4))
    return LZR_ERR_INVALID_ARG;
  if (launch_index(d_fp, n, 0, d_gidx, d_table, n_bins, bin_slots, d_index, d_unique, d_overflow,
                   (cudaStream_t)stream, &t_launches) != cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

int lzr_dedup_owner_counts(const uint8_t* d_fp, size_t n, uint32_t n_owners, uint32_t* d_counts,
                           lzr_stream_t stream) {
  t_launches = 0;
  if (n == 0) return LZR_OK;
  if (!d_fp || !d_counts || n_owners == 0 || !aligned(d_counts, 4)) return LZR_ERR_INVALID_ARG;
  if (launch_owner_counts(d_fp, n, n_owners, d_counts, (cudaStream_t)stream, &t_launches) !=
      cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

int lzr_dedup_route(const uint8_t* d_fp, size_t n, uint64_t first_chunk, uint32_t n_owners,
                    const uint64_t* d_base, uint32_t* d_cursor, uint8_t* d_send_fp,
                    uint64_t* d_send_gidx, uint32_t* d_slot, lzr_stream_t stream) {
  t_launches = 0;
  if (n == 0) return LZR_OK;
  if (!d_fp || !d_base || !d_cursor || !d_send_fp || !d_send_gidx || !d_slot || n_owners == 0)
    return LZR_ERR_INVALID_ARG;
  if (!aligned(d_base, 8) || !aligned(d_cursor, 4) || !aligned(d_send_gidx, 8) || !aligned(d_slot, 4))
    return LZR_ERR_INVALID_ARG;
  if (launch_route(d_fp, n, first_chunk, n_owners, d_base, d_cursor, d_send_fp, d_send_gidx, d_slot,
                   (cudaStream_t)stream, &t_launches) != cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

int lzr_dedup_unroute(const uint64_t* d_back, const uint32_t* d_slot, size_t n, uint64_t first_chunk,
                      uint64_t* d_index, uint32_t* d_unique, lzr_stream_t stream) {
  t_launches = 0;
  if (n == 0) return LZR_OK;
  if (!d_back || !d_slot || !d_index || !d_unique) return LZR_ERR_INVALID_ARG;
  if (!aligned(d_back, 8) || !aligned(d_slot, 4) || !aligned(d_index, 8) || !aligned(d_unique, 4))
    return LZR_ERR_INVALID_ARG;
  if (launch_unroute(d_back, d_slot, n, first_chunk, d_index, d_unique, (cudaStream_t)stream,
                     &t_launches) != cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

int lzr_gather_chunks(const void* d_in, size_t n_bytes, uint32_t chunk_size,
                      const uint32_t* d_unique, const uint64_t* d_rank, void* d_out,
                      lzr_stream_t stream) {
  t_launches = 0;
  if (n_bytes == 0) return LZR_OK;
  if (!d_in || !d_unique || !d_rank || !d_out || chunk_size == 0) return LZR_ERR_INVALID_ARG;
  if (!aligned(d_unique, 4) || !aligned(d_rank, 8)) return LZR_ERR_INVALID_ARG;
  DevInfo di;
  if (dev_info(&di) != cudaSuccess) return LZR_ERR_CUDA;
  if (launch_gather((const uint8_t*)d_in, n_bytes, chunk_size, d_unique, d_rank, (uint8_t*)d_out,
                    di.sm_count, (cudaStream_t)stream, &t_launches) != cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

size_t lzr_decompress_workspace_bytes(size_t n_bytes, const lzr_params* p) {
  if (lzr_validate_params(p) != LZR_OK) return 0;
  const size_t C = p->chunk_size;
  return align_up_z(decode_sched_bytes((n_bytes + C - 1) / C), 256);
}

int lzr_decompress_chunks(const void* d_comp, const uint32_t* d_sizes, const uint64_t* d_offsets,
                          size_t n_bytes, const lzr_params* p, void* d_out, int32_t* d_error,
                          void* d_workspace, size_t workspace_bytes, lzr_stream_t stream) {
  t_launches = 0;
  int st = lzr_validate_params(p);
  if (st) return st;
  cudaStream_t s = (cudaStream_t)stream;
  if (n_bytes && (!d_comp || !d_sizes || !d_offsets || !d_out)) return LZR_ERR_INVALID_ARG;
  if (d_error && !aligned(d_error, 4)) return LZR_ERR_INVALID_ARG;
  if (n_bytes && (!aligned(d_sizes, 4) || !aligned(d_offsets, 8))) return LZR_ERR_INVALID_ARG;
  DevInfo di;
  if (dev_info(&di) != cudaSuccess) return LZR_ERR_CUDA;
  if ((int)align_up(p->chunk_size, 16) > di.smem_optin)
    return LZR_ERR_UNSUPPORTED;
  uint32_t* sched = nullptr;  // the costliest-first schedule needs the workspace
  if (d_workspace) {
    if (!aligned(d_workspace, 4)) return LZR_ERR_INVALID_ARG;
    if (workspace_bytes < lzr_decompress_workspace_bytes(n_bytes, p)) return LZR_ERR_CAPACITY;
    sched = (uint32_t*)d_workspace;
  }
  if (launch_decode((const uint8_t*)d_comp, d_sizes, d_offsets, n_bytes, p->chunk_size,
                    p->min_match, (uint8_t*)d_out, d_error, di.sm_count, di.smem_optin, s,
                    &t_launches, 0, true, sched) != cudaSuccess)
    return LZR_ERR_CUDA;
  return LZR_OK;
}

// ---- host-buffer end-to-end pipeline ---------------------------------------

namespace {
struct HostSet {
  uint8_t *in, *out, *ws;
  uint32_t* sizes;
  uint64_t *offs, *total;
  size_t ws_bytes;
};

size_t set_bytes(size_t batch, const lzr_params* p) {
  const size_t C = p->chunk_size;
  const size_t N = (batch + C - 1) / C;
  return align_up_z(batch, 256) * 2 + align_up_z(4 * N, 256) + align_up_z(8 * N, 256) + 256 +
         ws_layout(batch, p).total;
}

HostSet carve(uint8_t* base, size_t batch, const lzr_params* p) {
  const size_t C = p->chunk_size;
  const size_t N = (batch + C - 1) / C;
  HostSet h;
  size_t o = 0;
  h.in = base + o; o += align_up_z(batch, 256);
  h.out = base + o; o += align_up_z(batch, 256);
  h.sizes = (uint32_t*)(base + o); o += align_up_z(4 * N, 256);
  h.offs = (uint64_t*)(base + o); o += align_up_z(8 * N, 256);
  h.total = (uint64_t*)(base + o); o += 256;
  h.ws = base + o;
  h.ws_bytes = ws_layout(batch, p).total;
  return h;
}
}  // namespace

// host_sets() buffer sets on as many streams: while batch b computes, earlier
// batches' compressed bytes go back (D2H) and later batches' inputs come in
// (H2D); a set is reused only after its D2H was issued on its own stream
// (stream order).
namespace {
constexpr int kMaxHostSets = 8;
// default 3 sets with shared copy streams (e2e sweep on 1 x B200, 256 MiB mix,
// PCIe 55 GB/s one way / 93 both ways, tools/e2e_sweep.py; 8/16/32 MiB batches):
// 3 sets 33.8/39.5/37.1 GB/s, 4 sets 37.6/38.6/36.4, 6 sets 35.6/36.0/32.6; a
// copy stream per set 33.0/37.4/37.0 (3 sets); H2D on the compute stream
// 32.6/37.0/36.5 (4 sets).  More sets split the link and the SMs over more
// batches at once, so each batch's bytes arrive later.  With the cached
// streams/events and launch attributes (no per-call / per-launch host setup):
// 3 sets 12/16/24 MiB 40.0/43.6/43.0, 4 sets 44.0/44.0/42.0, 5 sets 43.6/43.0/41.5
int host_sets() {  // LZR_HOST_SETS=2..8 overrides (tuning)
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("LZR_HOST_SETS");
    v = (e && *e >= '2' && *e <= '8') ? (*e - '0') : 3;
  }
  return v;
}

// copy-stream mode (LZR_HOST_SPLIT overrides, A/B): 0 = H2D on the set's
// compute stream; 1 = H2D on a copy stream per set; 2 = one H2D stream and one
// D2H stream shared by all sets (copies in batch order at full link rate)
int host_split() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("LZR_HOST_SPLIT");
    v = (e && *e >= '0' && *e <= '2') ? (*e - '0') : 2;
  }
  return v;
}

// Streams and events of the host pipeline.  Creating and destroying them on
// every call costs host time that the pipeline's first batches wait for, so
// each device keeps one cached set (created on first use, never destroyed;
// state is only these handles).  A call that finds its device's set in use
// (concurrent callers) creates a private set and destroys it afterwards.
struct HostStreams {
  cudaStream_t s[kMaxHostSets], cin[kMaxHostSets];
  cudaEvent_t ev_in[kMaxHostSets], ev_kdone[kMaxHostSets], ev_out[kMaxHostSets];
  int made = 0;       // sets created
  bool cached = false;
  bool busy = false;
};
constexpr int kMaxDevices = 64;
std::mutex g_hs_mu;
HostStreams g_hs[kMaxDevices];

bool make_host_streams(HostStreams* h, int n) {
  for (; h->made < n; ++h->made) {
    const int i = h->made;
    if (cudaStreamCreateWithFlags(&h->s[i], cudaStreamNonBlocking) != cudaSuccess) return false;
    if (cudaStreamCreateWithFlags(&h->cin[i], cudaStreamNonBlocking) != cudaSuccess) {
      cudaStreamDestroy(h->s[i]);
      return false;
    }
    cudaEvent_t* evs[3] = {&h->ev_in[i], &h->ev_kdone[i], &h->ev_out[i]};
    for (int e = 0; e < 3; ++e) {
      if (cudaEventCreateWithFlags(evs[e], cudaEventDisableTiming) != cudaSuccess) {
        for (int f = 0; f < e; ++f) cudaEventDestroy(*evs[f]);
        cudaStreamDestroy(h->s[i]);
        cudaStreamDestroy(h->cin[i]);
        return false;
      }
    }
  }
  return true;
}

void destroy_host_streams(HostStreams* h) {
  for (int i = 0; i < h->made; ++i) {
    cudaStreamDestroy(h->s[i]);
    cudaStreamDestroy(h->cin[i]);
    cudaEventDestroy(h->ev_in[i]);
    cudaEventDestroy(h->ev_kdone[i]);
    cudaEventDestroy(h->ev_out[i]);
  }
  h->made = 0;
}

HostStreams* acquire_host_streams(int n) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return nullptr;
  if (dev >= 0 && dev < kMaxDevices) {
    std::lock_guard<std::mutex> lk(g_hs_mu);
    HostStreams* h = &g_hs[dev];
    if (!h->busy) {
      if (!make_host_streams(h, n)) return nullptr;  // partial sets stay cached
      h->busy = true;
      h->cached = true;
      return h;
    }
  }
  HostStreams* h = new HostStreams();
  if (!make_host_streams(h, n)) {
    destroy_host_streams(h);
    delete h;
    return nullptr;
  }
  return h;
}

void release_host_streams(HostStreams* h) {
  if (h->cached) {
    std::lock_guard<std::mutex> lk(g_hs_mu);
    h->busy = false;
    return;
  }
  destroy_host_streams(h);
  delete h;
}
}  // namespace

size_t lzr_compress_host_scratch_bytes(size_t batch_bytes, const lzr_params* p) {
  if (lzr_validate_params(p) != LZR_OK || batch_bytes == 0) return 0;
  return host_sets() * align_up_z(set_bytes(batch_bytes, p), 256);
}

int lzr_compress_host(const void* h_in, size_t n_bytes, const lzr_params* p, void* h_out,
                      size_t out_capacity, uint32_t* h_sizes, uint64_t* h_offsets,
                      uint64_t* h_total, size_t batch_bytes, void* d_scratch,
                      size_t scratch_bytes) {
  int st = lzr_validate_params(p);
  if (st) return st;
  const size_t C = p->chunk_size;
  if (n_bytes == 0) {
    if (h_total) *h_total = 0;
    return LZR_OK;
  }
  if (!h_in || !h_out || !h_sizes || !h_offsets || !d_scratch) return LZR_ERR_INVALID_ARG;
  if (out_capacity < n_bytes) return LZR_ERR_CAPACITY;
  if (batch_bytes == 0) batch_bytes = align_up_z(n_bytes, C);
  if (batch_bytes % C) return LZR_ERR_INVALID_ARG;
  if (!aligned(d_scratch, 256)) return LZR_ERR_INVALID_ARG;
  const size_t per = align_up_z(set_bytes(batch_bytes, p), 256);
  const int kHostSets = host_sets();
  if (scratch_bytes < kHostSets * per) return LZR_ERR_CAPACITY;
  HostSet set[kMaxHostSets];
  for (int i = 0; i < kHostSets; ++i) set[i] = carve((uint8_t*)d_scratch + i * per, batch_bytes, p);
  // split (mode >= 1): a set's H2D waits only for the kernels of the set's
  // previous batch (its input buffer), not for that batch's D2H of compressed
  // bytes (which reads the output buffer; mode 2: the kernels wait for that)
  const int mode = host_split();
  const bool split = mode >= 1;
  // streams and events: the device's cached pool when free, else a private set
  HostStreams* hs = acquire_host_streams(kHostSets);
  if (!hs) return LZR_ERR_CUDA;
  cudaStream_t* s = hs->s;
  cudaStream_t* cin = hs->cin;
  cudaEvent_t* ev_in = hs->ev_in;
  cudaEvent_t* ev_kdone = hs->ev_kdone;
  cudaEvent_t* ev_out = hs->ev_out;
  const size_t nb = (n_bytes + batch_bytes - 1) / batch_bytes;
  const size_t chunks_per_batch = batch_bytes / C;
  uint64_t running = 0;
  int rc = LZR_OK;
  int launches = 0;
  auto issue = [&](size_t b) -> int {
    HostSet& h = set[b % kHostSets];
    cudaStream_t ss = s[b % kHostSets];
    const size_t lo = b * batch_bytes;
    const size_t len = n_bytes - lo < batch_bytes ? n_bytes - lo : batch_bytes;
    const size_t c0 = b * chunks_per_batch;
    const size_t N = (len + C - 1) / C;
    const int k = (int)(b % kHostSets);
    if (split) {
      cudaStream_t cs = mode == 2 ? cin[0] : cin[k];
      // h.in is free once the kernels of this set's previous batch are done
      if (b >= (size_t)kHostSets && cudaStreamWaitEvent(cs, ev_kdone[k], 0) != cudaSuccess)
        return LZR_ERR_CUDA;
      if (cudaMemcpyAsync(h.in, (const uint8_t*)h_in + lo, len, cudaMemcpyHostToDevice, cs) != cudaSuccess ||
          cudaEventRecord(ev_in[k], cs) != cudaSuccess || cudaStreamWaitEvent(ss, ev_in[k], 0) != cudaSuccess)
        return LZR_ERR_CUDA;
      // mode 2: h.out is free once the previous batch's bytes went back
      if (mode == 2 && b >= (size_t)kHostSets && cudaStreamWaitEvent(ss, ev_out[k], 0) != cudaSuccess)
        return LZR_ERR_CUDA;
    } else if (cudaMemcpyAsync(h.in, (const uint8_t*)h_in + lo, len, cudaMemcpyHostToDevice, ss) != cudaSuccess) {
      return LZR_ERR_CUDA;
    }
    int r = lzr_compress_chunks(h.in, len, p, h.out, batch_bytes, h.sizes, h.offs, h.total, h.ws,
                                h.ws_bytes, (lzr_stream_t)ss);
    if (r) return r;
    launches += t_launches;
    if (split && cudaEventRecord(ev_kdone[k], ss) != cudaSuccess) return LZR_ERR_CUDA;
    if (cudaMemcpyAsync(h_sizes + c0, h.sizes, 4 * N, cudaMemcpyDeviceToHost, ss) != cudaSuccess ||
        cudaMemcpyAsync(h_offsets + c0, h.offs, 8 * N, cudaMemcpyDeviceToHost, ss) != cudaSuccess)
      return LZR_ERR_CUDA;
    return LZR_OK;
  };
  auto finish = [&](size_t b) -> int {  // batch b's sizes are on the host: send its bytes back
    HostSet& h = set[b % kHostSets];
    cudaStream_t ss = s[b % kHostSets];
    if (cudaStreamSynchronize(ss) != cudaSuccess) return LZR_ERR_CUDA;
    const size_t lo = b * batch_bytes;
    const size_t len = n_bytes - lo < batch_bytes ? n_bytes - lo : batch_bytes;
    const size_t c0 = b * chunks_per_batch;
    const size_t N = (len + C - 1) / C;
    uint64_t tb = 0;  // batch total = sum of its sizes (already on the host)
    for (size_t i = 0; i < N; ++i) {
      h_offsets[c0 + i] += running;
      tb += h_sizes[c0 + i];
    }
    cudaStream_t ds = mode == 2 ? cin[1] : ss;
    if (tb && cudaMemcpyAsync((uint8_t*)h_out + running, h.out, tb, cudaMemcpyDeviceToHost, ds) != cudaSuccess)
      return LZR_ERR_CUDA;
    if (mode == 2 && cudaEventRecord(ev_out[b % kHostSets], ds) != cudaSuccess) return LZR_ERR_CUDA;
    running += tb;
    return LZR_OK;
  };
  // keep two batches in flight ahead of the one being finished
  for (size_t b = 0; b < nb && rc == LZR_OK; ++b) {
    rc = issue(b);
    if (rc == LZR_OK && b >= kHostSets - 1) rc = finish(b - (kHostSets - 1));
  }
  for (size_t b = nb > kHostSets - 1 ? nb - (kHostSets - 1) : 0; b < nb && rc == LZR_OK; ++b)
    rc = finish(b);
  for (int i = 0; i < kHostSets; ++i)
    if ((cudaStreamSynchronize(s[i]) != cudaSuccess || cudaStreamSynchronize(cin[i]) != cudaSuccess) &&
        rc == LZR_OK)
      rc = LZR_ERR_CUDA;
  release_host_streams(hs);
  if (h_total) *h_total = running;
  t_launches = launches;
  return rc;
}

}  // extern "C"

// ---- host-buffer decompression (the read path's end-to-end call) -----------

namespace {
struct DecSet {
  uint8_t *comp, *out;
  uint32_t* sizes;
  uint64_t* offs;
  uint32_t* sched;  // the batch's decode schedule
  int32_t* err;
};

size_t dec_set_bytes(size_t batch, const lzr_params* p) {
  const size_t C = p->chunk_size;
  const size_t N = (batch + C - 1) / C;
  return 2 * align_up_z(batch, 256) + align_up_z(4 * N, 256) + align_up_z(8 * N, 256) +
         align_up_z(decode_sched_bytes(N), 256) + 256;
}

DecSet dec_carve(uint8_t* base, size_t batch, const lzr_params* p) {
  const size_t C = p->chunk_size;
  const size_t N = (batch + C - 1) / C;
  DecSet d;
  size_t o = 0;
  d.comp = base + o; o += align_up_z(batch, 256);
  d.out = base + o; o += align_up_z(batch, 256);
  d.sizes = (uint32_t*)(base + o); o += align_up_z(4 * N, 256);
  d.offs = (uint64_t*)(base + o); o += align_up_z(8 * N, 256);
  d.sched = (uint32_t*)(base + o); o += align_up_z(decode_sched_bytes(N), 256);
  d.err = (int32_t*)(base + o);
  return d;
}
}  // namespace

extern "C" {

size_t lzr_decompress_host_scratch_bytes(size_t batch_bytes, const lzr_params* p) {
  if (lzr_validate_params(p) != LZR_OK || batch_bytes == 0) return 0;
  return host_sets() * align_up_z(dec_set_bytes(batch_bytes, p), 256);
}

int lzr_decompress_host(const void* h_comp, const uint32_t* h_sizes, const uint64_t* h_offsets,
                        size_t n_bytes, const lzr_params* p, void* h_out, int32_t* h_error,
                        size_t batch_bytes, void* d_scratch, size_t scratch_bytes) {
  int st = lzr_validate_params(p);
  if (st) return st;
  const size_t C = p->chunk_size;
  if (h_error) *h_error = 0;
  if (n_bytes == 0) return LZR_OK;
  if (!h_comp || !h_sizes || !h_offsets || !h_out || !d_scratch) return LZR_ERR_INVALID_ARG;
  if (batch_bytes == 0) batch_bytes = align_up_z(n_bytes, C);
  if (batch_bytes % C) return LZR_ERR_INVALID_ARG;
  if (!aligned(d_scratch, 256)) return LZR_ERR_INVALID_ARG;
  DevInfo di;
  if (dev_info(&di) != cudaSuccess) return LZR_ERR_CUDA;
  const size_t per = align_up_z(dec_set_bytes(batch_bytes, p), 256);
  const int nsets = host_sets();
  if (scratch_bytes < nsets * per) return LZR_ERR_CAPACITY;
  const size_t nb = (n_bytes + batch_bytes - 1) / batch_bytes;
  const size_t cpb = batch_bytes / C;
  HostStreams* hs = acquire_host_streams(nsets);
  if (!hs) return LZR_ERR_CUDA;
  // one H2D stream, one D2H stream (copies in batch order at full link rate),
  // a compute stream per buffer set; events order the reuse of a set's
  // buffers.  One error word for the whole call (set 0's), every batch's
  // kernel reporting global chunk indices (err_base), initialised before the
  // first decode and fixed up after the last.
  cudaStream_t h2d = hs->cin[0], d2h = nsets > 1 ? hs->cin[1] : hs->cin[0];
  int32_t* derr = dec_carve((uint8_t*)d_scratch, batch_bytes, p).err;
  int rc = LZR_OK;
  int launches = 0;
  if (decode_err_init(derr, hs->s[0]) != cudaSuccess || cudaEventRecord(hs->ev_in[0], hs->s[0]) != cudaSuccess)
    rc = LZR_ERR_CUDA;
  for (int k = 1; k < nsets && rc == LZR_OK; ++k)
    if (cudaStreamWaitEvent(hs->s[k], hs->ev_in[0], 0) != cudaSuccess) rc = LZR_ERR_CUDA;
  for (size_t b = 0; b < nb && rc == LZR_OK; ++b) {
    const int k = (int)(b % nsets);
    DecSet d = dec_carve((uint8_t*)d_scratch + k * per, batch_bytes, p);
    const size_t c0 = b * cpb;
    const size_t len = n_bytes - b * batch_bytes < batch_bytes ? n_bytes - b * batch_bytes : batch_bytes;
    const size_t N = (len + C - 1) / C;
    // the batch's compressed bytes: the span [lo, hi) of its chunks' streams
    // (any offsets are allowed; compacted streams always fit the buffer)
    uint64_t lo = ~0ull, hi = 0;
    for (size_t i = 0; i < N; ++i) {
      const uint64_t o = h_offsets[c0 + i], e = o + h_sizes[c0 + i];
      if (o < lo) lo = o;
      if (e > hi) hi = e;
    }
    if (hi - lo > batch_bytes) {
      rc = LZR_ERR_CAPACITY;
      break;
    }
    cudaStream_t ss = hs->s[k];
    // H2D once the set's previous decode has read its inputs
    if ((b >= (size_t)nsets && cudaStreamWaitEvent(h2d, hs->ev_kdone[k], 0) != cudaSuccess) ||
        (hi > lo && cudaMemcpyAsync(d.comp, (const uint8_t*)h_comp + lo, hi - lo, cudaMemcpyHostToDevice, h2d) != cudaSuccess) ||
        cudaMemcpyAsync(d.sizes, h_sizes + c0, 4 * N, cudaMemcpyHostToDevice, h2d) != cudaSuccess ||
        cudaMemcpyAsync(d.offs, h_offsets + c0, 8 * N, cudaMemcpyHostToDevice, h2d) != cudaSuccess ||
        cudaEventRecord(hs->ev_in[k], h2d) != cudaSuccess || cudaStreamWaitEvent(ss, hs->ev_in[k], 0) != cudaSuccess ||
        // the decode rewrites the set's output buffer once its previous D2H is done
        (b >= (size_t)nsets && cudaStreamWaitEvent(ss, hs->ev_out[k], 0) != cudaSuccess)) {
      rc = LZR_ERR_CUDA;
      break;
    }
    // offsets are the stream's own: the batch buffer stands at offset lo
    int l = 0;
    if (launch_decode(d.comp - lo, d.sizes, d.offs, len, (uint32_t)C, p->min_match, d.out, derr,
                      di.sm_count, di.smem_optin, ss, &l, c0, false, d.sched) != cudaSuccess ||
        cudaEventRecord(hs->ev_kdone[k], ss) != cudaSuccess || cudaStreamWaitEvent(d2h, hs->ev_kdone[k], 0) != cudaSuccess ||
        cudaMemcpyAsync((uint8_t*)h_out + b * batch_bytes, d.out, len, cudaMemcpyDeviceToHost, d2h) != cudaSuccess ||
        cudaEventRecord(hs->ev_out[k], d2h) != cudaSuccess) {
      rc = LZR_ERR_CUDA;
      break;
    }
    launches += l;
  }
  // every decode done -> fix the error word up and read it back
  for (int k = 0; k < nsets; ++k)
    if (cudaStreamSynchronize(hs->s[k]) != cudaSuccess && rc == LZR_OK) rc = LZR_ERR_CUDA;
  int32_t e_host = 0;
  if (rc == LZR_OK && (decode_err_fini(derr, hs->s[0], &launches) != cudaSuccess ||
                       cudaMemcpyAsync(&e_host, derr, 4, cudaMemcpyDeviceToHost, hs->s[0]) != cudaSuccess))
    rc = LZR_ERR_CUDA;
  if ((cudaStreamSynchronize(hs->s[0]) != cudaSuccess || cudaStreamSynchronize(h2d) != cudaSuccess ||
       cudaStreamSynchronize(d2h) != cudaSuccess) && rc == LZR_OK)
    rc = LZR_ERR_CUDA;
  release_host_streams(hs);
  if (h_error) *h_error = rc == LZR_OK ? e_host : 0;
  t_launches = launches;
  return rc;
}

}  // extern "C"
