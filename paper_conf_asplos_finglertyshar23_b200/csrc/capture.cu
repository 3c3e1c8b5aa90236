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

// Compact sort keys: (device << tb) | (time - tmin), with tb the bit width of the trace's
// time span and only as many 8-bit radix passes as the key's significant bits need (if that
// is odd, the sorted data ends in the _alt buffers and the consumers pick by its parity):
// the same order as the full 63-bit (device << 47 | time) key, in 4-6 passes instead of 8
// for traces spanning seconds.
struct KeyParams {
  unsigned long long tmin, tmax;  // over arrivals and completions (47-bit times)
  unsigned int dmax;              // largest device id (16 bits)
  int32_t tb;                     // time bits of the key
  int32_t npasses;                // radix passes of both sorts
};

__device__ __forceinline__ uint64_t ckey(const KeyParams &p, int32_t dev, int64_t t) {
  return ((uint64_t)(uint32_t)(dev & 0xFFFF) << p.tb) | (((uint64_t)t & kTimeMask) - p.tmin);
}

__global__ void key_range(const int64_t *__restrict__ a, const int64_t *__restrict__ c,
                          const int32_t *__restrict__ dev, int64_t n, KeyParams *p) {
  unsigned long long lo = ~0ull, hi = 0;
  unsigned int dm = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long ta = (uint64_t)a[i] & kTimeMask, tc = (uint64_t)c[i] & kTimeMask;
    lo = min(lo, min(ta, tc));
    hi = max(hi, max(ta, tc));
    if (dev) dm = max(dm, (unsigned int)(dev[i] & 0xFFFF));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
    dm = max(dm, __shfl_xor_sync(0xffffffffu, dm, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMin(&p->tmin, lo);
    atomicMax(&p->tmax, hi);
    atomicMax(&p->dmax, dm);
  }
}

__global__ void key_params(KeyParams *p) {
  const uint64_t span = p->tmax >= p->tmin ? p->tmax - p->tmin : 0;
  const int tb = span ? 64 - __clzll((long long)span) : 1;
  const int db = p->dmax ? 32 - __clz((int)p->dmax) : 0;
  const int passes = (tb + db + 7) / 8;
  p->tb = tb;
  p->npasses = passes;  // odd: the sorted data ends in the _alt buffers (consumers check)
}

__global__ void make_keys(const int64_t *__restrict__ a, const int64_t *__restrict__ c,
                          const int32_t *__restrict__ dev, int64_t n, uint64_t *ka, uint64_t *kc,
                          int32_t *ic, int32_t *ia, const KeyParams *__restrict__ pp) {
  const KeyParams p = *pp;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t d = dev ? dev[i] : 0;
    ka[i] = ckey(p, d, a[i]);
    kc[i] = ckey(p, d, c[i]);
    ic[i] = (int32_t)i;
    ia[i] = (int32_t)i;
  }
}

__global__ void invert(const int32_t *__restrict__ idx0, const int32_t *__restrict__ idx1,
                       int64_t n, int32_t *rank, const KeyParams *__restrict__ pp) {
  const int32_t *idx = (pp->npasses & 1) ? idx1 : idx0;  // where the sort left its result
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
                              int64_t n, const uint64_t *__restrict__ kc0,
                              const uint64_t *__restrict__ kc1,
                              const int32_t *__restrict__ rank_a, int32_t *q,
                              int64_t *ub_out, const KeyParams *__restrict__ pp) {
  const KeyParams p = *pp;
  const uint64_t *kc_sorted = (p.npasses & 1) ? kc1 : kc0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t d = dev ? dev[i] : 0;
    // device segment start: the smallest key of device d (time offset 0)
    const int64_t start = bsearch(kc_sorted, n, (uint64_t)(uint32_t)(d & 0xFFFF) << p.tb, false);
    const int64_t ub = bsearch(kc_sorted, n, ckey(p, d, a[i]), true);   // completions <= a_i
    q[i] = (int32_t)((rank_a[i] - start + 1) - (ub - start));
    ub_out[i] = ((int64_t)start << 32) | (ub - start);  // (segment start, completed count)
  }
}

__global__ void history(const int64_t *__restrict__ a, const int64_t *__restrict__ c,
                        int64_t n, const int32_t *__restrict__ idx_c0,
                        const int32_t *__restrict__ idx_c1,
                        const int32_t *__restrict__ q, const int64_t *__restrict__ ub_in,
                        uint32_t *__restrict__ raw, const KeyParams *__restrict__ pp) {
  const int32_t *idx_c = (pp->npasses & 1) ? idx_c1 : idx_c0;
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
  size_t ka, kc, ka2, kc2, iota, ia, ia2, ic, rank, q, ub, sort, kp, total;
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
  L.ia2 = o; o += a256(n * 4);  // the arrival sort's own alternate (odd pass counts)
  L.ic = o; o += a256(n * 4);
  L.rank = o; o += a256(n * 4);
  L.q = o; o += a256(n * 4);
  L.ub = o; o += a256(n * 8);
  L.sort = o; o += a256(sort_bytes);
  L.kp = o; o += a256(sizeof(KeyParams));
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
  KeyParams *kp = reinterpret_cast<KeyParams *>(b + L.kp);
  if (n <= 0) return cudaSuccess;
  // key range: tmin = all ones, tmax = dmax = 0, then atomics
  cudaError_t e = cudaMemsetAsync(kp, 0, sizeof(KeyParams), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(&kp->tmin, 0xFF, sizeof(kp->tmin), s);
  if (e != cudaSuccess) return e;
  key_range<<<grid, threads, 0, s>>>(a, c, dev, n, kp);
  key_params<<<1, 1, 0, s>>>(kp);
  make_keys<<<grid, threads, 0, s>>>(a, c, dev, n, U64(L.ka), U64(L.kc), I32(L.ic), I32(L.ia), kp);
  // (device, completion, index) and (device, arrival, index) orders; up to 8 passes of 8
  // bits, the device skipping the top ones the compact keys do not need (an even count), so
  // the results land back in kc / ic and ka / ia
  bool alt_c = false, alt_a = false;
  const int32_t *np = &kp->npasses;
  e = radix_sort_pairs(U64(L.kc), U64(L.kc2), I32(L.ic), I32(L.iota), n, kTimeBits + 16,
                       b + L.sort, s, &alt_c, np);
  if (e != cudaSuccess) return e;
  e = radix_sort_pairs(U64(L.ka), U64(L.ka2), I32(L.ia), I32(L.ia2), n, kTimeBits + 16,
                       b + L.sort, s, &alt_a, np);
  if (e != cudaSuccess) return e;
  // 8 host-side passes always end in kc / ic and ka / ia; the device ran kp->npasses of
  // them, so the consumers pick the buffers by its parity
  (void)alt_c;
  (void)alt_a;
  invert<<<grid, threads, 0, s>>>(I32(L.ia), I32(L.ia2), n, I32(L.rank), kp);
  pending_count<<<grid, threads, 0, s>>>(a, dev, n, U64(L.kc), U64(L.kc2), I32(L.rank), I32(L.q),
                                         reinterpret_cast<int64_t *>(b + L.ub), kp);
  history<<<grid, threads, 0, s>>>(a, c, n, I32(L.ic), I32(L.iota), I32(L.q),
                                   reinterpret_cast<const int64_t *>(b + L.ub), raw, kp);
  count_launch(6);
  return cudaGetLastError();
}

}  // namespace lake
