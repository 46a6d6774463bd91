// scan_compact.cu -- step a6: device-wide exclusive scan of the per-chunk sizes
// (single-pass decoupled look-back) and compaction of the chunk streams into
// one contiguous output in chunk order (R11).  The paper merged GPU results on
// the CPU (§3.2(2) "the CPU must refine the results"); here it stays on the
// device.  Both kernels are HBM/latency bound and tiny next to encode.
#include "lzr_internal.cuh"

namespace lzr {

namespace {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;  // 2048 sizes per tile

constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagPrefix = 2ull << 62;
constexpr uint64_t kValMask = (1ull << 62) - 1;

__device__ __forceinline__ uint64_t ld_status(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_status(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// ws: [0] u32 tile counter; [256..) u64 status per tile.  Zeroed before launch.
__global__ void __launch_bounds__(kScanThreads) lzr_scan_kernel(const uint32_t* __restrict__ sizes,
                                                               size_t n, uint64_t base,
                                                               const uint64_t* base_ptr,
                                                               uint64_t* __restrict__ offsets,
                                                               uint64_t* total, uint8_t* ws) {
  if (base_ptr) base += *base_ptr;  // device-side running base (chained batches)
  __shared__ uint32_t s_tile;
  __shared__ uint64_t s_warp[kScanThreads / 32];
  __shared__ uint64_t s_prefix;
  uint32_t* counter = reinterpret_cast<uint32_t*>(ws);
  uint64_t* status = reinterpret_cast<uint64_t*>(ws + 256);
  if (threadIdx.x == 0) s_tile = atomicAdd(counter, 1u);  // tiles in launch order: look-back progresses
  __syncthreads();
  const size_t tile = s_tile;
  const size_t t0 = tile * kScanTile + (size_t)threadIdx.x * kScanItems;
  uint32_t v[kScanItems];
  uint64_t local = 0;
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    v[k] = (t0 + k < n) ? sizes[t0 + k] : 0u;
    local += v[k];
  }
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  uint64_t incl = local;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t t = __shfl_up_sync(kFull, incl, o);
    if ((int)lane >= o) incl += t;
  }
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  uint64_t wbase = 0, agg = 0;
#pragma unroll
  for (int w = 0; w < kScanThreads / 32; ++w) {
    if (w < (int)warp) wbase += s_warp[w];
    agg += s_warp[w];
  }
  if (warp == 0) {
    uint64_t prefix = 0;
    if (tile == 0) {
      if (lane == 0) st_status(&status[0], kFlagPrefix | agg);
    } else {
      if (lane == 0) st_status(&status[tile], kFlagAgg | agg);
      // look back 32 predecessors at a time
      long j = (long)tile - 1;
      for (;;) {
        const long idx = j - (long)lane;
        uint64_t st = 0;
        if (idx >= 0) {
#ifdef LZR_WATCHDOG
          uint32_t spins = 0;
#endif
          do {
            LZR_SPIN_GUARD(spins, "scan look-back")
            st = ld_status(&status[idx]);
          } while ((st >> 62) == 0);
        } else {
          st = kFlagPrefix;  // before tile 0: prefix 0
        }
        const uint32_t pmask = __ballot_sync(kFull, (st >> 62) == 2);
        const uint32_t stop = pmask ? (uint32_t)(__ffs(pmask) - 1) : 32u;
        uint64_t contrib = (lane <= stop) ? (st & kValMask) : 0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) contrib += __shfl_xor_sync(kFull, contrib, o);
        prefix += contrib;
        if (pmask) break;
        j -= 32;
      }
      if (lane == 0) st_status(&status[tile], kFlagPrefix | (prefix + agg));
    }
    if (lane == 0) s_prefix = prefix;
  }
  __syncthreads();
  uint64_t run = base + s_prefix + wbase + (incl - local);
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    if (t0 + k < n) offsets[t0 + k] = run;
    run += v[k];
  }
  const size_t ntiles = (n + kScanTile - 1) / kScanTile;
  if (total && tile == ntiles - 1 && threadIdx.x == 0) *total = base + s_prefix + agg;
}

// Copy S bytes src -> dst (dst arbitrary alignment, src 16-byte aligned chunk
// base) with one warp: bytes up to a 16-byte boundary of dst, then 16-byte
// stores assembled from funnel-shifted source words (full-line writes also when
// dst is pinned host memory written over PCIe), then the byte tail.  Reads stay
// inside [src, src + S).
__device__ __forceinline__ void warp_copy(uint8_t* dst, const uint8_t* src, uint32_t S,
                                          uint32_t lane) {
  uint32_t head = (16u - (uint32_t)((uintptr_t)dst & 15u)) & 15u;
  if (head > S) head = S;
  if (lane < head) dst[lane] = src[lane];
  const uint32_t a = head & 3u;  // byte misalignment of the body's source
  const uint32_t sw = head >> 2;
  const uint32_t full = S >> 2;  // whole source words
  // 16-byte output vectors whose 4 (or 5 when misaligned) source words are whole
  long nv = ((long)S - (long)head) >> 4;
  const long lim = ((long)full - (long)sw - (a ? 1 : 0)) >> 2;
  if (nv > lim) nv = lim;
  if (nv < 0) nv = 0;
  const uint32_t* s32 = reinterpret_cast<const uint32_t*>(src);
  uint4* d128 = reinterpret_cast<uint4*>(dst + head);
  const uint32_t sh = a << 3;
  for (long k = lane; k < nv; k += 32) {
    const uint32_t w = sw + 4 * (uint32_t)k;
    const uint32_t w0 = s32[w], w1 = s32[w + 1], w2 = s32[w + 2], w3 = s32[w + 3];
    const uint32_t w4 = a ? s32[w + 4] : 0u;
    d128[k] = a ? make_uint4(__funnelshift_r(w0, w1, sh), __funnelshift_r(w1, w2, sh),
                             __funnelshift_r(w2, w3, sh), __funnelshift_r(w3, w4, sh))
                : make_uint4(w0, w1, w2, w3);
  }
  for (uint32_t i = head + (uint32_t)nv * 16u + lane; i < S; i += 32) dst[i] = src[i];
}

__global__ void __launch_bounds__(256) lzr_compact_kernel(const uint8_t* __restrict__ in,
                                                          size_t n_bytes, uint32_t C,
                                                          const uint8_t* __restrict__ slots,
                                                          size_t slot_stride,
                                                          const uint32_t* __restrict__ sizes,
                                                          const uint64_t* __restrict__ offsets,
                                                          uint8_t* __restrict__ out, size_t N) {
  const uint32_t lane = threadIdx.x & 31u;
  const size_t gw = ((size_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const size_t nw = ((size_t)gridDim.x * blockDim.x) >> 5;
  for (size_t i = gw; i < N; i += nw) {
    const size_t lo = i * C;
    const uint32_t ni = (uint32_t)min((size_t)C, n_bytes - lo);
    const uint32_t S = sizes[i];
    const uint8_t* src = (S == ni) ? in + lo : slots + i * slot_stride;  // raw: the input (R9)
    warp_copy(out + offsets[i], src, S, lane);
  }
}

}  // namespace

size_t scan_ws_bytes(size_t n) {
  const size_t ntiles = (n + kScanTile - 1) / kScanTile;
  return align_up_z(256 + ntiles * 8, 256);
}

cudaError_t launch_scan(const uint32_t* sizes, size_t n, uint64_t base, const uint64_t* base_ptr,
                        uint64_t* offsets, uint64_t* total, void* ws, cudaStream_t s,
                        int* launches) {
  cudaError_t err = cudaMemsetAsync(ws, 0, scan_ws_bytes(n), s);
  if (err != cudaSuccess) return err;
  const size_t ntiles = (n + kScanTile - 1) / kScanTile;
  if (ntiles == 0) return cudaSuccess;
  lzr_scan_kernel<<<(unsigned)ntiles, kScanThreads, 0, s>>>(sizes, n, base, base_ptr, offsets,
                                                            total, (uint8_t*)ws);
  if (launches) ++*launches;
  return cudaGetLastError();
}

cudaError_t launch_compact(const uint8_t* in, size_t n_bytes, uint32_t C, const uint8_t* slots,
                           size_t slot_stride, const uint32_t* sizes, const uint64_t* offsets, uint8_t* out,
                           int sm_count, cudaStream_t s, int* launches) {
  const size_t N = (n_bytes + C - 1) / C;
  if (N == 0) return cudaSuccess;
  size_t blocks = (N + 7) / 8;
  const size_t cap = (size_t)sm_count * 8;
  if (blocks > cap) blocks = cap;
  lzr_compact_kernel<<<(unsigned)blocks, 256, 0, s>>>(in, n_bytes, C, slots, slot_stride, sizes,
                                                     offsets, out, N);
  if (launches) ++*launches;
  return cudaGetLastError();
}

}  // namespace lzr
