// lzr_internal.cuh -- device helpers and launch plumbing shared by the sm_100a
// kernels of liblzr.so (encode, scan/compact, decode).  Part of the CUDA path
// only; the oracle (oracle/) shares nothing with it.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "../../include/lzr.h"

namespace lzr {

constexpr uint32_t kFull = 0xFFFFFFFFu;

__host__ __device__ constexpr uint32_t align_up(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }
__host__ __device__ constexpr size_t align_up_z(size_t x, size_t a) { return (x + a - 1) / a * a; }

// Unaligned little-endian 32-bit load from a shared-memory byte buffer whose
// base is 16-byte aligned: two aligned LDS.32 + one funnel shift.
__device__ __forceinline__ uint32_t ld32u(const uint8_t* base, uint32_t p) {
  const uint32_t* w = reinterpret_cast<const uint32_t*>(base);
  uint32_t a = w[p >> 2];
  uint32_t b = w[(p >> 2) + 1];
  return __funnelshift_r(a, b, (p & 3u) << 3);
}

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---- mbarrier + 1-D bulk TMA (cp.async.bulk) ---------------------------------
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void tma_bulk_g2s(void* smem_dst, const void* gmem_src, uint32_t bytes,
                                             uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(smem_dst)),
      "l"(gmem_src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
#ifdef LZR_WATCHDOG
#define LZR_SPIN_GUARD(cnt, what)                                                          \
  if (++(cnt) == (1u << 20)) {                                                             \
    printf("lzr watchdog: %s stuck, block %d thread %d\n", what, blockIdx.x, threadIdx.x); \
    __trap();                                                                              \
  }
#else
#define LZR_SPIN_GUARD(cnt, what)
#endif

__device__ __forceinline__ void mbar_wait_parity(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
#ifdef LZR_WATCHDOG
  uint32_t spins = 0;
#endif
  while (!done) {
    LZR_SPIN_GUARD(spins, "mbarrier wait")
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  }
}

// ---- encode kernel shared-memory layout (one region per group of K warps) ---
// run list capacity per chunk (runs of one byte value of length >= k): about
// one zero run per 128 bytes of chunk (the zero-runs class has one per ~300 B)
__host__ __device__ constexpr uint32_t enc_max_runs(uint32_t C) {
  const uint32_t r = (C / 128 + 7) & ~7u;
  return r < 24 ? 24 : r;
}

struct EncLayout {
  uint32_t K, nsplit, max_runs, off_sorted, off_slot, off_bm, off_mbar, per_group, hbits, bm_words, tb_words, fbits;
  // (no further fields: the kernels take EncArgs by value, and ptxas's register
  // allocation of the 4 KiB kernel was measured to change -- a spill -- with its size)
};

// Chunks above 32 KiB (up to the format's 64 KiB): one
// chunk's index no longer fits next to 15-bit positions and per-position slot
// arrays, so the big layout keeps full 16-bit positions in the index, bucket
// ends instead of bucket-start marks (B = 8192 buckets), no per-position slot
// array (a search finds p's own entry inside its bucket), and the K
// token-start bitmaps of the walk segments in the group's global scratch
// (L2-resident, next to the (d-1) scratch).
#ifndef LZR_BIG_CHUNK
#define LZR_BIG_CHUNK 32768
#endif
constexpr uint32_t kBigChunk = LZR_BIG_CHUNK;
#ifndef LZR_BIG_WARPS
#define LZR_BIG_WARPS 32u
#endif
constexpr uint32_t kBigHashBits = 13;

__host__ __device__ constexpr uint32_t enc_hash_bits(uint32_t C) {
  uint32_t hb = 0;
  while ((2u << hb) <= C && hb < 15) ++hb;  // largest power of two <= C (the table lives in 2C bytes)
  return hb;
}

// K warps per chunk; NS of them share the index scatter, each with its own
// cursor array, so NS * B u16 counters must fit the 2 max(C, B)-byte slot
// region: B = (largest power of two <= C) / NS
__host__ __device__ constexpr bool enc_big(uint32_t C) { return C > kBigChunk; }

__host__ __device__ constexpr EncLayout enc_layout(uint32_t C, uint32_t K, uint32_t NS) {
  EncLayout L{};
  L.K = K;
  const bool big = enc_big(C);
  L.hbits = big ? kBigHashBits : enc_hash_bits(C);
  L.nsplit = 1;
  while (L.nsplit < NS && L.hbits > 4) {  // (big: NS splits share the 8192 counters)
    --L.hbits;
    L.nsplit <<= 1;
  }
  L.fbits = 5;  // raw pre-filter: 2^fbits bits inside the 2C-byte index region (16C bits)
  while ((2u << L.fbits) <= 16 * C && L.fbits < 20) ++L.fbits;
  uint32_t B = 1u << L.hbits;
  // chunk bytes + 20 zero bytes: 16-byte compares read up to 19 bytes past n
  uint32_t o = align_up(C + 20, 4);
  L.off_sorted = o;
  o += 2 * C;  // u16 positions grouped by hash bucket, ascending
  L.off_slot = o;
  // u16 histogram -> cursors -> slot of each position (big: -> bucket ends)
  o += big ? 2 * B * L.nsplit : 2 * (C > B ? C : B);  // (NS cursor arrays of B counters)
  L.off_bm = o;
  L.bm_words = (C + 31) / 32 + 1;  // candidate / byte-change: +1 for two-word funnel reads
  L.tb_words = (C + 31) / 32;      // per-segment token-start bitmaps
  // candidate, byte-change, K token-start bitmaps (big: in global scratch); run
  // list; ctrl (4 + 2K words)
  L.max_runs = enc_max_runs(C);
  const bool tbg = big || K >= 16;  // walk bitmaps in the global scratch
  o += 4 * (2 * L.bm_words + (tbg ? 0 : K * L.tb_words) + L.max_runs + 4 + 2 * K + (C + 1023) / 1024);
  o = align_up(o, 8);
  L.off_mbar = o;
  o += 8;
  L.per_group = align_up(o, 16);  // next group's chunk buffer: 16-byte aligned (TMA)
  return L;
}

// global scratch bytes per resident group: (d-1) per position (u16), + the K
// token-start bitmaps when big
__host__ __device__ inline size_t enc_scratch_per_group(const EncLayout& L, uint32_t C) {
  return (enc_big(C) || L.K >= 16) ? align_up_z(2 * (size_t)C + 4 * (size_t)L.K * L.tb_words, 256)
                                   : 2 * (size_t)C;
}

struct EncArgs {
  const uint8_t* in;
  size_t n_bytes;
  uint32_t N;  // chunks (fits: N <= 2^32 - 1 checked on host)
  uint32_t C, W, m, M;
  uint32_t lazy;           // parse rule: 0 greedy (R8), 1 one-step lazy (R21)
  uint32_t kbytes, kmask;  // candidate key = first min(m,4) bytes
  EncLayout L;
  uint8_t* slots;    // workspace: chunk i's stream at slots + i*C
  uint8_t* scratch;  // workspace: 2C bytes per resident group (u16 (d-1) per position)
  uint32_t* sizes;
  uint32_t* counter;  // work distribution, zeroed before launch
};

// ---- workspace layout ---------------------------------------------------------
struct WsLayout {
  size_t ctrl_off, slots_off, scratch_off, scan_off, total;
};
constexpr uint32_t kMaxGroupsPerSm = 16;  // scratch bound: resident groups per SM
constexpr uint32_t kSmemPerSm = 233472;   // shared memory per SM (228 KB)
size_t scan_ws_bytes(size_t n);
WsLayout ws_layout(size_t n_bytes, const lzr_params* p);

// launches (defined in the .cu files); return cudaError_t of the launch
cudaError_t launch_encode(const EncArgs& a, int sm_count, int smem_optin, cudaStream_t s, int* launches);
cudaError_t launch_scan(const uint32_t* sizes, size_t n, uint64_t base, const uint64_t* base_ptr,
                        uint64_t* offsets, uint64_t* total, void* ws, cudaStream_t s,
                        int* launches);
cudaError_t launch_compact(const uint8_t* in, size_t n_bytes, uint32_t C, const uint8_t* slots,
                           size_t slot_stride,
                           const uint32_t* sizes, const uint64_t* offsets, uint8_t* out,
                           int sm_count, cudaStream_t s, int* launches);
// decode: err (optional) receives min(1 + err_base + chunk) over corrupt
// chunks; err_own: this launch initialises it (0x7F7F7F7F) and fixes it up to
// 0 when nothing was corrupt -- otherwise the caller does both
// (decode_err_init / decode_err_fini) around several launches sharing it
cudaError_t launch_decode(const uint8_t* comp, const uint32_t* sizes, const uint64_t* offsets,
                          size_t n_bytes, uint32_t C, uint32_t m, uint8_t* out, int32_t* err,
                          int sm_count, int smem_optin, cudaStream_t s, int* launches,
                          uint64_t err_base = 0, bool err_own = true, uint32_t* sched = nullptr);
// decode schedule workspace (costliest chunks first): 128 counters + N indices
inline size_t decode_sched_bytes(size_t N) { return (128 + N) * sizeof(uint32_t); }
cudaError_t decode_err_init(int32_t* err, cudaStream_t s);
cudaError_t decode_err_fini(int32_t* err, cudaStream_t s, int* launches);

// dedup.cu
cudaError_t launch_sha1(const uint8_t* in, size_t n, uint32_t C, uint8_t* fp, cudaStream_t s,
                        int* launches);
size_t dedup_entry_bytes();
cudaError_t launch_index(const uint8_t* fps, size_t N, uint64_t first, const uint64_t* gidx,
                         void* table, uint32_t n_bins, uint32_t bin_slots, uint64_t* index,
                         uint32_t* unique, uint32_t* overflow, cudaStream_t s, int* launches);
cudaError_t launch_owner_counts(const uint8_t* fps, size_t N, uint32_t n_owners, uint32_t* counts,
                                cudaStream_t s, int* launches);
cudaError_t launch_route(const uint8_t* fps, size_t N, uint64_t first, uint32_t n_owners,
                         const uint64_t* base, uint32_t* cursor, uint8_t* send_fp, uint64_t* send_gidx,
                         uint32_t* slot, cudaStream_t s, int* launches);
cudaError_t launch_unroute(const uint64_t* back, const uint32_t* slot, size_t N, uint64_t first,
                           uint64_t* index, uint32_t* unique, cudaStream_t s, int* launches);
cudaError_t launch_gather(const uint8_t* in, size_t n, uint32_t C, const uint32_t* unique,
                          const uint64_t* rank, uint8_t* out, int sm_count, cudaStream_t s,
                          int* launches);

}  // namespace lzr
