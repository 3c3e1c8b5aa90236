// capture.cu — GPU feature capture: the raw LinnOS records the
// feature registry would have captured on issue / completion (Fig. 4/5),
// computed for a whole trace at once instead of I/O by I/O in the block layer.
//
// For I/O i of device d (arrival a_i, completion c_i, ns), readings R7-R10:
//   q_now_i   = pending I/Os of d at issue including i
//             = (rank of (a_i, i) among d's arrivals) + 1 - #{ j of d : c_j <= a_i }
//   history   = the 4 largest (c_j, j) with c_j <= a_i, newest first;
//               lat_us = floor((c_j - a_j)/1000), q_hist = q_now_j, missing -> 0
// (every j with c_j <= a_i arrived strictly before i, so the completed count needs no
// arrival condition).
//
// Device algorithm: two stable LSD radix sorts (sort.cu, hand-written) of 63-bit keys
// (device << 47 | time) with I/O indices as values — completions and arrivals, both ordered
// by (device, time, index) — then one thread per I/O: a binary search of (device << 47 | a_i)
// in the sorted completions gives the completed count and the newest four completed I/Os.
#include "lake_internal.h"

namespace lake {
namespace {

constexpr int kTimeBits = 47;
constexpr uint64_t kTimeMask = (1ull << kTimeBits) - 1;

__device__ __forceinline__ uint64_t ckey(int32_t dev, int64_t t) {
  return ((uint64_t)(uint32_t)(dev & 0xFFFF) << kTimeBits) | ((uint64_t)t & kTimeMask);
}

__global__ void make_keys(const int64_t *__restrict__ a, const int64_t *__restrict__ c,
                          const int32_t *__restrict__ dev, int64_t n, uint64_t *ka, uint64_t *kc,
                          int32_t *ic, int32_t *ia) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t d = dev ? dev[i] : 0;
    ka[i] = ckey(d, a[i]);
    kc[i] = ckey(d, c[i]);
    ic[i] = (int32_t)i;
    ia[i] = (int32_t)i;
  }
}

__global__ void invert(const int32_t *__restrict__ idx, int64_t n, int32_t *rank) {
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    rank[idx[p]] = (int32_t)p;
}

// first position p in [0, n) with keys[p] >= x (lower) or > x (upper)
__device__ __forceinline__ int64_t bsearch(const uint64_t *__restrict__ keys, int64_t n,
                                           uint64_t x, bool upper) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    const uint64_t k = keys[mid];
    if (upper ? (k <= x) : (k < x)) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

__global__ void pending_count(const int64_t *__restrict__ a, const int32_t *__restrict__ dev,
                              int64_t n, const uint64_t *__restrict__ kc_sorted,
                              const int32_t *__restrict__ rank_a, int32_t *q,
                              int64_t *ub_out) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t d = dev ? dev[i] : 0;
    const int64_t start = bsearch(kc_sorted, n, ckey(d, 0), false);  // device segment start
    const int64_t ub = bsearch(kc_sorted, n, ckey(d, a[i]), true);   // completions <= a_i
    q[i] = (int32_t)((rank_a[i] - start + 1) - (ub - start));
    ub_out[i] = ((int64_t)start << 32) | (ub - start);  // (segment start, completed count)
  }
}

__global__ void history(const int64_t *__restrict__ a, const int64_t *__restrict__ c,
                        int64_t n, const int32_t *__restrict__ idx_c,
                        const int32_t *__restrict__ q, const int64_t *__restrict__ ub_in,
                        uint32_t *__restrict__ raw) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t start = ub_in[i] >> 32, cnt = ub_in[i] & 0xFFFFFFFFll;
    uint32_t r[9];
    r[0] = (uint32_t)q[i];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      if (k < cnt) {
        const int32_t j = idx_c[start + cnt - 1 - k];
        const int64_t us = (c[j] - a[j]) / 1000;
        r[1 + k] = us > 0xFFFFFFFFll ? 0xFFFFFFFFu : (uint32_t)us;
        r[5 + k] = (uint32_t)q[j];
      } else {
        r[1 + k] = 0;
        r[5 + k] = 0;
      }
    }
#pragma unroll
    for (int f = 0; f < 9; ++f) raw[i * 9 + f] = r[f];
  }
}

size_t a256(size_t x) { return (x + 255) & ~(size_t)255; }

struct CapLayout {
  size_t ka, kc, ka2, kc2, iota, ia, ic, rank, q, ub, sort, total;
};

CapLayout cap_layout(int64_t n, size_t sort_bytes) {
  CapLayout L{};
  size_t o = 0;
  L.ka = o; o += a256(n * 8);
  L.kc = o; o += a256(n * 8);
  L.ka2 = o; o += a256(n * 8);
  L.kc2 = o; o += a256(n * 8);
  L.iota = o; o += a256(n * 4);
  L.ia = o; o += a256(n * 4);
  L.ic = o; o += a256(n * 4);
  L.rank = o; o += a256(n * 4);
  L.q = o; o += a256(n * 4);
  L.ub = o; o += a256(n * 8);
  L.sort = o; o += a256(sort_bytes);
  L.total = o;
  return L;
}

}  // namespace

size_t capture_workspace_bytes(int64_t n) {
  return cap_layout(n, radix_sort_workspace_bytes(n)).total;
}

cudaError_t launch_capture(const int64_t *a, const int64_t *c, const int32_t *dev, int64_t n,
                           uint32_t *raw, void *ws, size_t ws_bytes, cudaStream_t s) {
  const CapLayout L = cap_layout(n, radix_sort_workspace_bytes(n));
  if (ws_bytes < L.total) return cudaErrorMemoryAllocation;
  uint8_t *b = static_cast<uint8_t *>(ws);
  auto U64 = [&](size_t off) { return reinterpret_cast<uint64_t *>(b + off); };
  auto I32 = [&](size_t off) { return reinterpret_cast<int32_t *>(b + off); };
  const int threads = 256;
  const int grid = (int)((n + threads - 1) / threads < 148 * 16 ? (n + threads - 1) / threads
                                                                : 148 * 16);
  make_keys<<<grid, threads, 0, s>>>(a, c, dev, n, U64(L.ka), U64(L.kc), I32(L.ic), I32(L.ia));
  // (device, completion, index) and (device, arrival, index) orders; 8 passes of 8 bits,
  // so the results land back in kc / ic and ka / ia
  bool alt_c = false, alt_a = false;
  cudaError_t e = radix_sort_pairs(U64(L.kc), U64(L.kc2), I32(L.ic), I32(L.iota), n,
                                   kTimeBits + 16, b + L.sort, s, &alt_c);
  if (e != cudaSuccess) return e;
  e = radix_sort_pairs(U64(L.ka), U64(L.ka2), I32(L.ia), I32(L.iota), n, kTimeBits + 16,
                       b + L.sort, s, &alt_a);
  if (e != cudaSuccess) return e;
  const uint64_t *kc_sorted = alt_c ? U64(L.kc2) : U64(L.kc);
  const int32_t *idx_c = alt_c ? I32(L.iota) : I32(L.ic);
  const int32_t *idx_a = alt_a ? I32(L.iota) : I32(L.ia);
  static_assert((kTimeBits + 16 + 7) / 8 % 2 == 0, "even pass count: results in place");
  invert<<<grid, threads, 0, s>>>(idx_a, n, I32(L.rank));
  pending_count<<<grid, threads, 0, s>>>(a, dev, n, kc_sorted, I32(L.rank), I32(L.q),
                                         reinterpret_cast<int64_t *>(b + L.ub));
  history<<<grid, threads, 0, s>>>(a, c, n, idx_c, I32(L.q),
                                   reinterpret_cast<const int64_t *>(b + L.ub), raw);
  count_launch(4);
  return cudaGetLastError();
}

}  // namespace lake
