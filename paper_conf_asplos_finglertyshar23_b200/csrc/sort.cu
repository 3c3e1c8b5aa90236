// sort.cu — stable LSD radix sort of (u64 key, i32 value) pairs, hand-written for the
// GPU feature capture (capture.cu; it orders completions and arrivals by (device, time,
// index)). Replaces the round-1 library sort (CUB onesweep).
//
// One pass per 8-bit digit, four kernels each:
//   rs_count    per 2,048-key tile: digit histogram (shared atomics) -> counts[digit][tile]
//               (digit-major, so that one exclusive scan of the array gives every
//               (digit, tile) its output base in stable order)
//   rs_scan_*   exclusive scan of counts (per 4,096-entry block, then the block sums)
//   rs_scatter  per tile: each warp ranks its 256 consecutive keys in 8 in-order rounds of 32
//               (__match_any_sync groups equal digits; rank = warp count so far + earlier
//               lanes), per-digit prefixes over warps and digits give every key its position
//               in the tile's sorted order; the tile is re-ordered in shared memory and written
//               out as contiguous runs per digit (coalesced)
// Stability: within a tile, keys of equal digit keep (warp, round, lane) = input order; across
// tiles the digit-major scan puts earlier tiles first.
#include <cstdint>

#include "lake_internal.h"

namespace lake {
namespace {

constexpr int kRsThreads = 256;
constexpr int kRsWarps = kRsThreads / 32;
constexpr int kRsItems = 8;                        // keys per thread (8 rounds of 32 per warp)
constexpr int kRsTile = kRsThreads * kRsItems;     // 2,048 keys per tile
constexpr int kRsBits = 8;                         // digit width: 8 passes for 63-bit keys
constexpr int kRsBins = 1 << kRsBits;
constexpr int kRsScanBlock = 4096;                 // entries per scan block (1,024 x 4)
static_assert(kRsBins == kRsThreads, "one thread per digit in the per-tile scans");

__device__ __forceinline__ uint32_t digit_of(uint64_t k, int shift) {
  return (uint32_t)(k >> shift) & (kRsBins - 1);
}

__global__ void __launch_bounds__(kRsThreads)
rs_count(const uint64_t *__restrict__ keys, int64_t n, int shift, int32_t *__restrict__ counts,
         int64_t ntiles, const int32_t *__restrict__ npasses) {
  if (npasses && shift / kRsBits >= *npasses) return;  // a skipped (all-zero) digit
  __shared__ int32_t bins[kRsBins];
  bins[threadIdx.x] = 0;
  __syncthreads();
  const int64_t base = (int64_t)blockIdx.x * kRsTile;
#pragma unroll 4
  for (int j = 0; j < kRsItems; ++j) {  // coalesced
    const int64_t i = base + (int64_t)j * kRsThreads + threadIdx.x;
    if (i < n) atomicAdd(&bins[digit_of(__ldg(keys + i), shift)], 1);
  }
  __syncthreads();
  counts[(int64_t)threadIdx.x * ntiles + blockIdx.x] = bins[threadIdx.x];
}

// exclusive scan of 1,024 values held one per thread (1,024 threads)
__device__ __forceinline__ int32_t block_scan1024(int32_t v, int32_t *wsum, int32_t *total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[w] = x;
  __syncthreads();
  if (w == 0) {
    int32_t t = wsum[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t y = __shfl_up_sync(0xffffffffu, t, o);
      if (lane >= o) t += y;
    }
    wsum[lane] = t;
    if (lane == 31) *total = t;
  }
  __syncthreads();
  const int32_t r = x - v + (w > 0 ? wsum[w - 1] : 0);
  __syncthreads();
  return r;
}

// in place: each 4,096-entry block of `a` -> its exclusive scan; bsum[block] = block total
__global__ void __launch_bounds__(1024)
rs_scan_blocks(int32_t *__restrict__ a, int64_t m, int32_t *__restrict__ bsum, int pass,
               const int32_t *__restrict__ npasses) {
  if (npasses && pass >= *npasses) return;
  __shared__ int32_t wsum[32], total;
  const int64_t i0 = (int64_t)blockIdx.x * kRsScanBlock + 4 * threadIdx.x;
  int32_t v[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) v[j] = i0 + j < m ? a[i0 + j] : 0;
  const int32_t s = v[0] + v[1] + v[2] + v[3];
  int32_t run = block_scan1024(s, wsum, &total);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    if (i0 + j < m) a[i0 + j] = run;
    run += v[j];
  }
  if (threadIdx.x == 0) bsum[blockIdx.x] = total;
}

// one block: bsum[0..nb) -> exclusive scan, in place (loops over 1,024-entry pieces)
__global__ void __launch_bounds__(1024) rs_scan_sums(int32_t *__restrict__ bsum, int64_t nb,
                                                     int pass, const int32_t *__restrict__ npasses) {
  if (npasses && pass >= *npasses) return;
  __shared__ int32_t wsum[32], total;
  int32_t carry = 0;
  for (int64_t b0 = 0; b0 < nb; b0 += 1024) {
    const int64_t i = b0 + threadIdx.x;
    const int32_t v = i < nb ? bsum[i] : 0;
    const int32_t r = block_scan1024(v, wsum, &total);
    if (i < nb) bsum[i] = carry + r;
    carry += total;
    __syncthreads();
  }
}

__global__ void __launch_bounds__(kRsThreads)
rs_scatter(const uint64_t *__restrict__ kin, const int32_t *__restrict__ vin, int64_t n, int shift,
           const int32_t *__restrict__ offs, const int32_t *__restrict__ bsum, int64_t ntiles,
           uint64_t *__restrict__ kout, int32_t *__restrict__ vout,
           const int32_t *__restrict__ npasses) {
  if (npasses && shift / kRsBits >= *npasses) return;
  __shared__ uint64_t sk[kRsTile];
  __shared__ int32_t sv[kRsTile];
  __shared__ int32_t whist[kRsWarps][kRsBins];  // per-warp digit counts -> prefix over warps
  __shared__ int32_t tstart[kRsBins];           // digit start within the sorted tile
  __shared__ int32_t gbase[kRsBins];            // digit start in the output
  __shared__ int32_t wsum[kRsWarps];
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  const int64_t base = (int64_t)blockIdx.x * kRsTile;
  const int cnt = (int)((n - base) < kRsTile ? (n - base) : kRsTile);
#pragma unroll
  for (int ww = 0; ww < kRsWarps; ++ww) whist[ww][t] = 0;
  {
    const int64_t e = (int64_t)t * ntiles + blockIdx.x;
    gbase[t] = offs[e] + bsum[e / kRsScanBlock];
  }
  __syncthreads();
  // warp w ranks keys [w*256, w*256 + 256) of the tile in 8 rounds of 32, in order: a key's
  // rank among its warp's keys of the same digit = earlier rounds' count + earlier lanes
  uint64_t k[kRsItems];
  int32_t v[kRsItems], lr[kRsItems];
  const uint32_t lt = (1u << lane) - 1;
#pragma unroll
  for (int r = 0; r < kRsItems; ++r) {
    const int q = w * (32 * kRsItems) + r * 32 + lane;
    const bool ok = q < cnt;
    k[r] = ok ? __ldg(kin + base + q) : 0ull;
    v[r] = ok ? __ldg(vin + base + q) : 0;
  }
#pragma unroll
  for (int r = 0; r < kRsItems; ++r) {
    const int q = w * (32 * kRsItems) + r * 32 + lane;
    const bool ok = q < cnt;
    const uint32_t d = ok ? digit_of(k[r], shift) : kRsBins;  // padding: its own group
    const uint32_t peers = __match_any_sync(0xffffffffu, d);
    lr[r] = ok ? whist[w][d] + __popc(peers & lt) : 0;
    __syncwarp();
    if (ok && (peers & lt) == 0) whist[w][d] += __popc(peers);  // group leader
    __syncwarp();
  }
  __syncthreads();
  // thread t = digit t: exclusive prefix of its counts over warps, then over digits
  int32_t run = 0;
#pragma unroll
  for (int ww = 0; ww < kRsWarps; ++ww) {
    const int32_t c = whist[ww][t];
    whist[ww][t] = run;
    run += c;
  }
  int32_t x = run;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[w] = x;
  __syncthreads();
  int32_t wpre = 0;
#pragma unroll
  for (int j = 0; j < kRsWarps; ++j) wpre += j < w ? wsum[j] : 0;
  tstart[t] = wpre + x - run;
  __syncthreads();
  // every key -> its position in the tile's stable sorted order (shared memory)
#pragma unroll
  for (int r = 0; r < kRsItems; ++r) {
    const int q = w * (32 * kRsItems) + r * 32 + lane;
    if (q < cnt) {
      const uint32_t d = digit_of(k[r], shift);
      const int p = tstart[d] + whist[w][d] + lr[r];
      sk[p] = k[r];
      sv[p] = v[r];
    }
  }
  __syncthreads();
  // contiguous runs per digit: sorted position p of digit d goes to gbase[d] + p - tstart[d]
  for (int p = t; p < cnt; p += kRsThreads) {
    const uint64_t kk = sk[p];
    const uint32_t d = digit_of(kk, shift);
    const int64_t pos = (int64_t)gbase[d] + (p - tstart[d]);
    kout[pos] = kk;
    vout[pos] = sv[p];
  }
}

int64_t rs_tiles(int64_t n) { return (n + kRsTile - 1) / kRsTile; }
int64_t rs_scan_blocks_of(int64_t n) { return (kRsBins * rs_tiles(n) + kRsScanBlock - 1) / kRsScanBlock; }

}  // namespace

size_t radix_sort_workspace_bytes(int64_t n) {
  return (size_t)(kRsBins * rs_tiles(n) + rs_scan_blocks_of(n) + 64) * sizeof(int32_t);
}

// Sorts (keys, vals) by the low `bits` bits of the keys, stably, ping-ponging with the _alt
// buffers; returns in *in_alt whether the result ended in the _alt buffers (odd pass count).
// d_npasses (device, optional): passes [*d_npasses, ceil(bits / 8)) are skipped on the device
// (their digits are zero in every key: a stable no-op); with an even *d_npasses and an even
// pass count the result still lands in the input buffers.
cudaError_t radix_sort_pairs(uint64_t *keys, uint64_t *keys_alt, int32_t *vals, int32_t *vals_alt,
                             int64_t n, int bits, void *ws, cudaStream_t s, bool *in_alt,
                             const int32_t *d_npasses) {
  *in_alt = false;
  if (n <= 0) return cudaSuccess;
  if (n > (int64_t)INT32_MAX) return cudaErrorInvalidValue;
  const int64_t nt = rs_tiles(n), m = kRsBins * nt, nsb = rs_scan_blocks_of(n);
  int32_t *counts = static_cast<int32_t *>(ws);
  int32_t *bsum = counts + m;
  uint64_t *ka = keys, *kb = keys_alt;
  int32_t *va = vals, *vb = vals_alt;
  for (int shift = 0; shift < bits; shift += kRsBits) {
    const int pass = shift / kRsBits;
    rs_count<<<(unsigned)nt, kRsThreads, 0, s>>>(ka, n, shift, counts, nt, d_npasses);
    rs_scan_blocks<<<(unsigned)nsb, 1024, 0, s>>>(counts, m, bsum, pass, d_npasses);
    rs_scan_sums<<<1, 1024, 0, s>>>(bsum, nsb, pass, d_npasses);
    rs_scatter<<<(unsigned)nt, kRsThreads, 0, s>>>(ka, va, n, shift, counts, bsum, nt, kb, vb,
                                                   d_npasses);
    count_launch(4);
    uint64_t *tk = ka; ka = kb; kb = tk;
    int32_t *tv = va; va = vb; vb = tv;
    *in_alt = !*in_alt;
  }
  return cudaGetLastError();
}

}  // namespace lake
