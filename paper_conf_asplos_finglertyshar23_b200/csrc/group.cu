// group.cu — model grouping for lake_linnos_infer_multi: one feature registry (hence one
// model) per block device (Fig. 4 caption); batches from several
// devices arrive interleaved and are scored per model (score_features).
//
// Counting sort of I/O indices by model id, on the device:
//   group_hist     per-chunk SMEM histogram -> one global atomic per (chunk, model), and the
//                  chunk histogram stored for the scatter
//   group_scan     one block: exclusive scans of counts and of tiles per model (for both
//                  the 64-row FP32 tiles and the 256-row tensor-core tiles)
//   group_scatter  stored chunk histogram -> reserve a range per model -> positions
//   group_tiles    one thread per tile: binary search of its model, begin, count
// Unknown ids (out of range or not loaded) go to the tail of perm; lake_linnos_multi_grouped
// writes decision 0 / NaN logits for them. Results do not depend on the order inside a
// model's range (every row is computed independently), so the scatter need not be stable.
#include <atomic>
#include <cstddef>
#include <type_traits>

#include "digitize.cuh"
#include "lake_internal.h"
#include "lake_ptx.cuh"

namespace lake {
namespace {

constexpr int kGBlock = 512;
#ifndef LAKE_GCHUNK
#define LAKE_GCHUNK 4096
#endif
constexpr int kChunk = LAKE_GCHUNK;  // I/Os per block-iteration in hist/scatter
constexpr int kBins = LAKE_MAX_MODELS + 1;  // model slots + "unknown"

struct WsHeader {
  int32_t counts[LAKE_MAX_MODELS];
  int32_t cursor_unused[LAKE_MAX_MODELS];  // (cursors live in WsLayout::cursor, padded)
  int32_t offsets[LAKE_MAX_MODELS];
  int32_t tile_off64[LAKE_MAX_MODELS + 1];
  int32_t tile_off256[LAKE_MAX_MODELS + 1];  // by rank in ord256 (NN models first)
  int32_t ord256[LAKE_MAX_MODELS];           // rank -> model slot
  int32_t n_tiles64;
  int32_t n_tiles256;
  int32_t n_tiles256_nn;                     // the NN models' tiles: [0, n_tiles256_nn)
  int32_t n_known;
  int32_t unk_cursor;
  int64_t n_unknown;
  int32_t arch_mask;
  int32_t pad;
  // "model slot is loaded", snapshotted once per call by group_init: histogram and scatter
  // must classify every id identically even if another thread loads / unloads a model id
  // (not used by this call's known models) meanwhile; a divergent view would overrun a
  // model's reserved range of perm
  uint8_t known[LAKE_MAX_MODELS];
  uint8_t nnc[LAKE_MAX_MODELS];  // ... and holds an NN model (one hidden layer), same snapshot
};

__host__ __device__ inline size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

constexpr int kCursorStride = 32;  // int32 per cursor (128 B)

struct WsLayout {
  size_t cursor, header, perm, t64_model, t64_begin, t64_count, t256_model, t256_begin, t256_count,
      chunk_counts, pdig, total;
  int64_t max64, max256;
};

WsLayout ws_layout(int64_t n) {
  WsLayout L{};
  L.max64 = group_max_tiles(n, kF32TileM);
  L.max256 = group_max_tiles(n, kTcTileRows);
  size_t off = 0;
  L.header = off; off = align256(off + sizeof(WsHeader));
  L.perm = off; off = align256(off + (size_t)n * 4);
  L.t64_model = off; off = align256(off + (size_t)L.max64 * 4);
  L.t64_begin = off; off = align256(off + (size_t)L.max64 * 8);
  L.t64_count = off; off = align256(off + (size_t)L.max64 * 4);
  L.t256_model = off; off = align256(off + (size_t)L.max256 * 4);
  L.t256_begin = off; off = align256(off + (size_t)L.max256 * 8);
  L.t256_count = off; off = align256(off + (size_t)L.max256 * 4);
  // per-chunk histograms written by group_hist, read back by group_scatter (no recount)
  L.chunk_counts = off; off = align256(off + (size_t)((n + kChunk - 1) / kChunk) * kBins * 4);
  // per-model scatter cursors, one 128-B line each: every chunk reserves its range of each
  // model with a global atomic, and 64 models' cursors packed into 2 lines serialised ~130K
  // atomics on those lines (the scatter ran at half of HBM bandwidth)
  L.cursor = off; off = align256(off + (size_t)kBins * kCursorStride * 4);
  // packed digit rows (16 B per I/O) in model-grouped order, for the tensor-core kernel's
  // contiguous bulk-copy staging
  L.pdig = off; off = align256(off + (size_t)n * 16);
  L.total = off;
  return L;
}

__device__ __forceinline__ bool known(const DevModel *table, int32_t m) {
  return m >= 0 && m < LAKE_MAX_MODELS && table[m].arch >= 0;
}

// Per-block SMEM copy of the call's snapshot of "model slot is loaded", so the per-I/O test
// is a shared-memory byte read instead of a dependent global load.
__device__ __forceinline__ void load_known(const WsHeader *h, uint8_t *known_s) {
  for (int m = threadIdx.x; m < LAKE_MAX_MODELS; m += blockDim.x) known_s[m] = h->known[m];
}

// Packed digit row of I/O i of the caller's input.
template <int IN_KIND>
__device__ __forceinline__ uint4 pack_input(const void *in, int64_t i) {
  if constexpr (IN_KIND == LAKE_IN_RAW) {
    const uint32_t *src = static_cast<const uint32_t *>(in) + i * 9;
    uint32_t rec[9];
#pragma unroll
    for (int f = 0; f < 9; ++f) rec[f] = __ldg(src + f);
    return pack_record(rec);
  } else {
    const uint4 *src = reinterpret_cast<const uint4 *>(static_cast<const uint8_t *>(in) + i * 32);
    return pack_digit_bytes(__ldg(src), __ldg(src + 1));
  }
}

// Zero the header and snapshot the device model table (one thread per model slot).
__global__ void __launch_bounds__(LAKE_MAX_MODELS)
group_init(const DevModel *__restrict__ table, WsHeader *h) {
  uint32_t *w = reinterpret_cast<uint32_t *>(h);
  for (uint32_t i = threadIdx.x; i < offsetof(WsHeader, known) / 4; i += blockDim.x) w[i] = 0;
  h->known[threadIdx.x] = table[threadIdx.x].arch >= 0 ? 1 : 0;
  h->nnc[threadIdx.x] = (table[threadIdx.x].arch >= 0 && table[threadIdx.x].nh == 1) ? 1 : 0;
}
__device__ __forceinline__ int32_t bin_of(const uint8_t *known_s, int32_t m) {
  return ((unsigned)m < (unsigned)LAKE_MAX_MODELS && known_s[m]) ? m : LAKE_MAX_MODELS;
}

template <typename IdT>
__global__ void __launch_bounds__(kGBlock)
group_hist(const IdT *__restrict__ ids, int64_t n, WsHeader *h,
           int32_t *__restrict__ chunk_counts) {
  __shared__ int32_t cnt[LAKE_MAX_MODELS + 1];
  __shared__ uint8_t known_s[LAKE_MAX_MODELS];
  load_known(h, known_s);
  for (int64_t base = (int64_t)blockIdx.x * kChunk; base < n; base += (int64_t)gridDim.x * kChunk) {
    for (int i = threadIdx.x; i <= LAKE_MAX_MODELS; i += kGBlock) cnt[i] = 0;
    __syncthreads();
    const int64_t end = (base + kChunk) < n ? base + kChunk : n;
    if (sizeof(IdT) == 4 && end - base == kChunk && (reinterpret_cast<uintptr_t>(ids) & 15) == 0) {
      // full chunk of 16-B-aligned int32 ids: 16-B loads, all of the thread's in flight at once
      constexpr int V = kChunk / (4 * kGBlock);
      int4 v[V];
#pragma unroll
      for (int u = 0; u < V; ++u)
        v[u] = __ldg(reinterpret_cast<const int4 *>(ids + base) + threadIdx.x + u * kGBlock);
#pragma unroll
      for (int u = 0; u < V; ++u) {
        atomicAdd(&cnt[bin_of(known_s, v[u].x)], 1);
        atomicAdd(&cnt[bin_of(known_s, v[u].y)], 1);
        atomicAdd(&cnt[bin_of(known_s, v[u].z)], 1);
        atomicAdd(&cnt[bin_of(known_s, v[u].w)], 1);
      }
    } else
    for (int64_t i0 = base + threadIdx.x; i0 < end; i0 += 4 * kGBlock) {
      int32_t idv[4];  // four loads in flight per thread
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int64_t i = i0 + (int64_t)u * kGBlock;
        idv[u] = i < end ? (int32_t)__ldg(ids + i) : 0;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (i0 + (int64_t)u * kGBlock < end) atomicAdd(&cnt[bin_of(known_s, idv[u])], 1);
    }
    __syncthreads();
    int32_t *cc = chunk_counts + (base / kChunk) * kBins;
    for (int m = threadIdx.x; m < kBins; m += kGBlock) cc[m] = cnt[m];
    for (int m = threadIdx.x; m < LAKE_MAX_MODELS; m += kGBlock)
      if (cnt[m]) atomicAdd(&h->counts[m], cnt[m]);
    if (threadIdx.x == 0 && cnt[LAKE_MAX_MODELS])
      atomicAdd((unsigned long long *)&h->n_unknown, (unsigned long long)cnt[LAKE_MAX_MODELS]);
    __syncthreads();
  }
}

// exclusive block scan over 1024 values (1024 threads)
__device__ int32_t block_excl_scan(int32_t v, int32_t *warp_tot, int32_t *total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_tot[w] = x;
  __syncthreads();
  if (w == 0) {
    int32_t t = warp_tot[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t y = __shfl_up_sync(0xffffffffu, t, o);
      if (lane >= o) t += y;
    }
    warp_tot[lane] = t;  // inclusive over warps
    if (lane == 31) *total = t;
  }
  __syncthreads();
  const int32_t r = x - v + (w > 0 ? warp_tot[w - 1] : 0);
  __syncthreads();
  return r;
}

__global__ void __launch_bounds__(LAKE_MAX_MODELS)
group_scan(WsHeader *h, int32_t *cursor) {
  __shared__ int32_t warp_tot[32];
  __shared__ int32_t total;
  const int m = threadIdx.x;
  const int32_t c = h->counts[m];
  const int32_t off = block_excl_scan(c, warp_tot, &total);
  h->offsets[m] = off;
  cursor[m * kCursorStride] = off;
  const int32_t n_known = total;
  const int32_t t64 = block_excl_scan((c + kF32TileM - 1) / kF32TileM, warp_tot, &total);
  h->tile_off64[m] = t64;
  const int32_t tot64 = total;
  // tensor-core tiles: NN models' first (slot order within each class), so that the NN tiles
  // form the prefix [0, n_tiles256_nn) that the NN kernel takes (api.cu: multi-model calls
  // mixing NN with NN+1/NN+2 run one kernel per class)
  const bool nn = h->nnc[m] != 0;
  const int32_t tc = (c + kTcTileRows - 1) / kTcTileRows;
  const int32_t t_nn = block_excl_scan(nn ? tc : 0, warp_tot, &total);
  const int32_t tot_nn = total;
  const int32_t t_ot = block_excl_scan(nn ? 0 : tc, warp_tot, &total);
  const int32_t tot256 = tot_nn + total;
  const int32_t r_nn = block_excl_scan(nn ? 1 : 0, warp_tot, &total);
  const int32_t rank = nn ? r_nn : total + (m - r_nn);
  h->ord256[rank] = m;
  h->tile_off256[rank] = nn ? t_nn : tot_nn + t_ot;
  if (m == 0) {
    h->n_known = n_known;
    cursor[LAKE_MAX_MODELS * kCursorStride] = n_known;
    h->n_tiles64 = tot64;
    h->n_tiles256 = tot256;
    h->n_tiles256_nn = tot_nn;
    h->tile_off64[LAKE_MAX_MODELS] = tot64;
    h->tile_off256[LAKE_MAX_MODELS] = tot256;
  }
}

// in_kind < 0: perm only; LAKE_IN_RAW / LAKE_IN_DIGITS: also the packed digit row of every
// known I/O at its grouped position (the I/O's input is read in arrival order: coalesced).
template <typename IdT, int IN_KIND>
__global__ void __launch_bounds__(kGBlock)
group_scatter(const IdT *__restrict__ ids, int64_t n, WsHeader *h, int32_t *__restrict__ perm,
              const int32_t *__restrict__ chunk_counts, const void *__restrict__ in,
              uint4 *__restrict__ pdig, int32_t *__restrict__ cursor) {
  __shared__ int32_t cnt[LAKE_MAX_MODELS + 1];
  __shared__ int32_t basep[LAKE_MAX_MODELS + 1];
  __shared__ uint8_t known_s[LAKE_MAX_MODELS];
  load_known(h, known_s);
  for (int64_t base = (int64_t)blockIdx.x * kChunk; base < n; base += (int64_t)gridDim.x * kChunk) {
    const int32_t *cc = chunk_counts + (base / kChunk) * kBins;  // this chunk's histogram
    for (int i = threadIdx.x; i < kBins; i += kGBlock) cnt[i] = cc[i];
    __syncthreads();
    const int64_t end = (base + kChunk) < n ? base + kChunk : n;
    for (int m = threadIdx.x; m <= LAKE_MAX_MODELS; m += kGBlock) {
      const int32_t c = cnt[m];
      if (c) basep[m] = atomicAdd(&cursor[m * kCursorStride], c);
      cnt[m] = 0;
    }
    __syncthreads();
    for (int64_t i = base + threadIdx.x; i < end; i += kGBlock) {
      const int32_t m = bin_of(known_s, (int32_t)__ldg(ids + i));
      const int32_t r = atomicAdd(&cnt[m], 1);
      perm[basep[m] + r] = (int32_t)i;
      if constexpr (IN_KIND >= 0) {
        if (m < LAKE_MAX_MODELS) pdig[basep[m] + r] = pack_input<IN_KIND>(in, i);
      }
    }
    __syncthreads();
  }
}

// multi_grouped after a separate multi_group call: packed rows gathered through perm
template <int IN_KIND>
__global__ void __launch_bounds__(256)
group_pack(const WsHeader *__restrict__ h, const int32_t *__restrict__ perm,
           const void *__restrict__ in, uint4 *__restrict__ pdig) {
  const int64_t nk = h->n_known;
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < nk;
       p += (int64_t)gridDim.x * blockDim.x)
    pdig[p] = pack_input<IN_KIND>(in, perm[p]);
}

// Scatter + packing (tensor-core paths), coalesced: a chunk's I/Os are first counting-sorted
// by model in shared memory (packed row, I/O index, model), then written out as contiguous
// per-model runs, so the 16-B packed-row and 4-B perm stores of a warp land in a few runs
// instead of ~25 scattered lines (the per-I/O scatter ran at 2.25 TB/s).
#ifndef LAKE_SCATTER_U
#define LAKE_SCATTER_U 2
#endif
#ifndef LAKE_SCATTER_PREFETCH
#define LAKE_SCATTER_PREFETCH 0
#endif
constexpr bool kScatterPrefetch = LAKE_SCATTER_PREFETCH;  // next iteration's loads issued early
constexpr int kScatterU = LAKE_SCATTER_U;  // records in flight per thread in the sort phase
constexpr int kWarpRaw = 32 * 36 / 16;       // 72 uint4: one warp's 32 consecutive raw records
constexpr size_t kPackSmem = (size_t)kChunk * (16 + 4) + (size_t)(kGBlock / 32) * kWarpRaw * 16;
static_assert(kChunk <= 65536, "chunk-relative index packed in 16 bits");

// Raw records of the warp's 32 consecutive I/Os [wb, wb+32): read as 72 coalesced 16-B loads
// (instead of 9 strided 4-B loads per lane, 9 L1 wavefronts each), passed through a per-warp
// shared buffer, and each lane takes back its own 36-B record (stride 9 words: conflict-free).
struct WarpRaw {
  uint4 v[3];
  __device__ __forceinline__ void load(const void *in, int64_t wb, int lane) {
    const uint4 *src = reinterpret_cast<const uint4 *>(static_cast<const uint8_t *>(in) + wb * 36);
    v[0] = __ldg(src + lane);
    v[1] = __ldg(src + 32 + lane);
    if (lane < kWarpRaw - 64) v[2] = __ldg(src + 64 + lane);
  }
  __device__ __forceinline__ uint4 pack(uint4 *stage, int lane) const {
    stage[lane] = v[0];
    stage[32 + lane] = v[1];
    if (lane < kWarpRaw - 64) stage[64 + lane] = v[2];
    __syncwarp();
    const uint32_t *w = reinterpret_cast<const uint32_t *>(stage) + lane * 9;
    uint32_t rec[9];
#pragma unroll
    for (int f = 0; f < 9; ++f) rec[f] = w[f];
    __syncwarp();
    return pack_record(rec);
  }
};

// One iteration's loads (kScatterU records per thread), held in registers until consumed.
template <typename IdT, int IN_KIND>
struct ScatterPrefetch {
  int32_t idv[kScatterU];
  WarpRaw wr[kScatterU];  // warp-staged raw records, or the packed row in wr[u].v[0]
  bool staged[kScatterU];
  __device__ __forceinline__ void issue(const IdT *ids, const void *in, int64_t c, int64_t end,
                                        int w, int lane, bool raw16) {
#pragma unroll
    for (int u = 0; u < kScatterU; ++u) {
      const int64_t wb = c + (int64_t)u * kGBlock + 32 * w, i = wb + lane;
      idv[u] = i < end ? (int32_t)__ldg(ids + i) : 0;
      staged[u] = IN_KIND == LAKE_IN_RAW && raw16 && wb + 32 <= end;
      if (staged[u]) wr[u].load(in, wb, lane);
      else wr[u].v[0] = i < end ? pack_input<IN_KIND>(in, i) : make_uint4(0, 0, 0, 0);
    }
  }
  __device__ __forceinline__ uint4 take(int u, uint4 *stage, int lane) const {
    return staged[u] ? wr[u].pack(stage, lane) : wr[u].v[0];
  }
};

template <typename IdT, int IN_KIND>
__global__ void __launch_bounds__(kGBlock, 2)
group_scatter_pack(const IdT *__restrict__ ids, int64_t n, WsHeader *h, int32_t *__restrict__ perm,
                   const int32_t *__restrict__ chunk_counts, const void *__restrict__ in,
                   uint4 *__restrict__ pdig, int32_t *__restrict__ cursor) {
  __shared__ int32_t cnt[kBins];    // chunk histogram, then per-model ranks
  __shared__ int32_t loff[kBins];   // exclusive scan of the chunk histogram
  __shared__ int32_t basep[kBins];  // reserved global base per model
  __shared__ int32_t wsum[kGBlock / 32];
  __shared__ uint8_t known_s[LAKE_MAX_MODELS];
  extern __shared__ __align__(16) uint8_t dyn[];
  uint4 *srow = reinterpret_cast<uint4 *>(dyn);                             // [kChunk] rows
  uint32_t *skey = reinterpret_cast<uint32_t *>(dyn + (size_t)kChunk * 16);  // model<<16 | i-base
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint4 *stage = reinterpret_cast<uint4 *>(dyn + (size_t)kChunk * 20) + w * kWarpRaw;
  const bool raw16 = IN_KIND == LAKE_IN_RAW && (reinterpret_cast<uintptr_t>(in) & 15) == 0;
  load_known(h, known_s);
  ScatterPrefetch<IdT, IN_KIND> pf;
  if (kScatterPrefetch && (int64_t)blockIdx.x * kChunk < n) {
    const int64_t b = (int64_t)blockIdx.x * kChunk;
    pf.issue(ids, in, b, (b + kChunk) < n ? b + kChunk : n, w, lane, raw16);
  }
  for (int64_t base = (int64_t)blockIdx.x * kChunk; base < n; base += (int64_t)gridDim.x * kChunk) {
    const int32_t *cc = chunk_counts + (base / kChunk) * kBins;
    const int64_t end = (base + kChunk) < n ? base + kChunk : n;
    // exclusive scan of the 1025 bins: thread t owns bins 2t, 2t+1 (t = 511 also bin 1024)
    const int b0 = 2 * threadIdx.x;
    const int32_t c0 = cc[b0], c1 = cc[b0 + 1], c2 = threadIdx.x == kGBlock - 1 ? cc[kBins - 1] : 0;
    int32_t x = c0 + c1 + c2;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[w] = x;
    __syncthreads();
    int32_t wpre = 0;
    for (int j = 0; j < w; ++j) wpre += wsum[j];
    const int32_t excl = wpre + x - (c0 + c1 + c2);
    loff[b0] = excl;
    loff[b0 + 1] = excl + c0;
    if (threadIdx.x == kGBlock - 1) loff[kBins - 1] = excl + c0 + c1;
    // reserve each model's run in the global grouping
    for (int m = threadIdx.x; m < kBins; m += kGBlock) {
      const int32_t c = cc[m];
      if (c) basep[m] = atomicAdd(&cursor[m * kCursorStride], c);
      cnt[m] = 0;
    }
    __syncthreads();
    // 1) counting sort into shared memory (input read in arrival order: coalesced); every
    // thread runs the same iterations (the warp-staged raw path synchronises the warp). The
    // loads of the next iteration (or of the next chunk's first one) are issued before this
    // iteration's shared-memory work, so they are in flight across the scan / reservation /
    // write-out phases instead of exposing a full DRAM latency per iteration.
    for (int64_t c = base; c < end; c += kScatterU * kGBlock) {
      uint4 pk[kScatterU];
      int32_t idc[kScatterU];
      if (!kScatterPrefetch) pf.issue(ids, in, c, end, w, lane, raw16);
#pragma unroll
      for (int u = 0; u < kScatterU; ++u) {
        idc[u] = pf.idv[u];
        pk[u] = pf.take(u, stage, lane);
      }
      int64_t nc = c + kScatterU * kGBlock, nend = end;
      if (nc >= end) {
        nc = base + (int64_t)gridDim.x * kChunk;
        nend = (nc + kChunk) < n ? nc + kChunk : n;
      }
      if (kScatterPrefetch && nc < n) pf.issue(ids, in, nc, nend, w, lane, raw16);
#pragma unroll
      for (int u = 0; u < kScatterU; ++u) {
        const int64_t i = c + (int64_t)u * kGBlock + threadIdx.x;
        if (i >= end) continue;
        const int32_t m = bin_of(known_s, idc[u]);
        const int32_t lp = loff[m] + atomicAdd(&cnt[m], 1);
        srow[lp] = pk[u];
        skey[lp] = ((uint32_t)m << 16) | (uint32_t)(i - base);
      }
    }
    __syncthreads();
    // 2) contiguous per-model runs out
    const int nk = (int)(end - base);
    for (int k = threadIdx.x; k < nk; k += kGBlock) {
      const uint32_t e = skey[k];
      const int m = (int)(e >> 16);
      const int32_t pos = basep[m] + (k - loff[m]);
      perm[pos] = (int32_t)(base + (e & 0xFFFFu));
      if (m < LAKE_MAX_MODELS) pdig[pos] = srow[k];
    }
    __syncthreads();
  }
}

// The same scatter + packing for raw records with 16-B-aligned records and ids, fed by bulk
// copies (cp.async.bulk, TMA engine) instead of per-warp loads: one block of 512 threads per
// SM streams its chunks' records and ids as 1,024-I/O sub-chunks (36 KB + ids) through a
// kTmaStages-deep shared-memory ring, so DRAM reads stay in flight across the per-chunk
// scan / reservation / write-out phases (the load-based kernel above exposed a DRAM latency
// per iteration: long-scoreboard stalls, 50% of HBM peak). Sorting, reservation and the
// per-model runs are those of group_scatter_pack.
#ifndef LAKE_SCATTER_TMA
#define LAKE_SCATTER_TMA 1
#endif
constexpr int kSub = 1024;                     // I/Os per bulk-copied sub-chunk
constexpr int kTmaStages = 3;
constexpr int kSubsPerChunk = kChunk / kSub;
static_assert(kChunk % kSub == 0 && kSub == 2 * kGBlock, "two records per thread per sub-chunk");
constexpr size_t kSubRawBytes = (size_t)kSub * 36;
constexpr size_t kSubIdBytes = (size_t)kSub * 4;   // room for int32 ids
constexpr size_t kTmaSmem = (size_t)kChunk * (16 + 4) + kTmaStages * (kSubRawBytes + kSubIdBytes);

template <typename IdT>
__global__ void __launch_bounds__(kGBlock, 1)
group_scatter_pack_tma(const IdT *__restrict__ ids, int64_t n, WsHeader *h,
                       int32_t *__restrict__ perm, const int32_t *__restrict__ chunk_counts,
                       const void *__restrict__ in, uint4 *__restrict__ pdig,
                       int32_t *__restrict__ cursor) {
  __shared__ int32_t cnt[kBins];
  __shared__ int32_t loff[kBins];
  __shared__ int32_t basep[kBins];
  __shared__ int32_t wsum[kGBlock / 32];
  __shared__ uint8_t known_s[LAKE_MAX_MODELS];
  __shared__ __align__(8) uint64_t full[kTmaStages];
  extern __shared__ __align__(16) uint8_t dyn[];
  uint4 *srow = reinterpret_cast<uint4 *>(dyn);
  uint32_t *skey = reinterpret_cast<uint32_t *>(dyn + (size_t)kChunk * 16);
  uint8_t *ring = dyn + (size_t)kChunk * 20;  // [stage] raw records | ids
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint8_t *raw = static_cast<const uint8_t *>(in);
  const int64_t G = gridDim.x;
  // sub-chunk q of this block: chunk blockIdx.x + (q / kSubsPerChunk) G, part q % kSubsPerChunk
  auto sub_base = [&](int64_t q) {
    return ((int64_t)blockIdx.x + (q / kSubsPerChunk) * G) * kChunk + (q % kSubsPerChunk) * kSub;
  };
  auto issue = [&](int64_t q) {  // thread 0: bring sub-chunk q into its ring stage
    const int64_t sb = sub_base(q);
    if (sb >= n) return;
    const int st = (int)(q % kTmaStages);
    const int64_t c = (n - sb) < kSub ? (n - sb) : kSub;
    const uint32_t rb = (uint32_t)(c * 36) & ~15u, ib = (uint32_t)(c * sizeof(IdT)) & ~15u;
    const uint32_t fb = ptx::smem_u32(&full[st]);
    uint8_t *dst = ring + (size_t)st * (kSubRawBytes + kSubIdBytes);
    ptx::mbar_arrive_expect_tx(fb, rb + ib);
    if (rb) ptx::bulk_g2s(ptx::smem_u32(dst), raw + sb * 36, rb, fb);
    if (ib) ptx::bulk_g2s(ptx::smem_u32(dst + kSubRawBytes), ids + sb, ib, fb);
  };
  if (threadIdx.x == 0) {
    for (int i = 0; i < kTmaStages; ++i) ptx::mbar_init(ptx::smem_u32(&full[i]), 1);
    ptx::fence_mbar_init();
  }
  load_known(h, known_s);
  __syncthreads();
  if (threadIdx.x == 0)
    for (int i = 0; i < kTmaStages; ++i) issue(i);
  int64_t q = 0;  // next sub-chunk to consume
  // The chunk histogram loads and the cursor reservations (global atomics with a returned
  // value) of chunk k+1 are issued during chunk k - loads before its sort phase, atomics
  // before its write-out - so neither round trip sits between two chunks.
  const int t = threadIdx.x;
  int32_t ns[3], nc[3], rv[3];  // next chunk: scan inputs (bins 2t, 2t+1, 1024), counts and
                                // reserved bases of bins t, t+512, t+1024
  auto load_next = [&](int64_t b) {
    const int32_t *cc = chunk_counts + (b / kChunk) * kBins;
    ns[0] = cc[2 * t];
    ns[1] = cc[2 * t + 1];
    ns[2] = t == kGBlock - 1 ? cc[kBins - 1] : 0;
#pragma unroll
    for (int i = 0; i < 3; ++i) nc[i] = (t + i * kGBlock < kBins) ? cc[t + i * kGBlock] : 0;
  };
  auto reserve_next = [&]() {
#pragma unroll
    for (int i = 0; i < 3; ++i)
      rv[i] = nc[i] ? atomicAdd(&cursor[(t + i * kGBlock) * kCursorStride], nc[i]) : 0;
  };
  if ((int64_t)blockIdx.x * kChunk < n) {
    load_next((int64_t)blockIdx.x * kChunk);
    reserve_next();
  }
  for (int64_t base = (int64_t)blockIdx.x * kChunk; base < n; base += G * kChunk) {
    const int64_t end = (base + kChunk) < n ? base + kChunk : n;
    const int64_t nbase = base + G * kChunk;
    const int b0 = 2 * t;
    const int32_t c0 = ns[0], c1 = ns[1], c2 = ns[2];
    int32_t x = c0 + c1 + c2;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[w] = x;
    __syncthreads();
    int32_t wpre = 0;
    for (int j = 0; j < w; ++j) wpre += wsum[j];
    const int32_t excl = wpre + x - (c0 + c1 + c2);
    loff[b0] = excl;
    loff[b0 + 1] = excl + c0;
    if (t == kGBlock - 1) loff[kBins - 1] = excl + c0 + c1;
#pragma unroll
    for (int i = 0; i < 3; ++i)
      if (t + i * kGBlock < kBins) {
        basep[t + i * kGBlock] = rv[i];
        cnt[t + i * kGBlock] = 0;
      }
    __syncthreads();
    if (nbase < n) load_next(nbase);
    // 1) counting sort of the chunk's sub-chunks, each read from its ring stage
    for (int64_t sb = base; sb < end; sb += kSub, ++q) {
      const int st = (int)(q % kTmaStages);
      const int64_t c = (end - sb) < kSub ? (end - sb) : kSub;
      const uint32_t rb = (uint32_t)(c * 36) & ~15u, ib = (uint32_t)(c * sizeof(IdT)) & ~15u;
      const uint8_t *sraw = ring + (size_t)st * (kSubRawBytes + kSubIdBytes);
      const IdT *sid = reinterpret_cast<const IdT *>(sraw + kSubRawBytes);
      ptx::mbar_wait(ptx::smem_u32(&full[st]), (uint32_t)((q / kTmaStages) & 1));
      auto sort_one = [&](int r, const uint32_t (&rec)[9], int32_t id) {
        const uint4 pk = pack_record(rec);
        const int32_t m = bin_of(known_s, id);
        const int32_t lp = loff[m] + atomicAdd(&cnt[m], 1);
        srow[lp] = pk;
        skey[lp] = ((uint32_t)m << 16) | (uint32_t)(sb + r - base);
      };
      if (c == kSub) {  // full sub-chunk (all but the call's last): shared memory only
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int r = threadIdx.x + u * kGBlock;
          uint32_t rec[9];
          const uint32_t *src = reinterpret_cast<const uint32_t *>(sraw) + r * 9;  // conflict-free
#pragma unroll
          for (int f = 0; f < 9; ++f) rec[f] = src[f];
          sort_one(r, rec, (int32_t)sid[r]);
        }
      } else {
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int r = threadIdx.x + u * kGBlock;
          if (r >= c) continue;
          uint32_t rec[9];
          if ((uint32_t)(r + 1) * 36 <= rb) {
            const uint32_t *src = reinterpret_cast<const uint32_t *>(sraw) + r * 9;
#pragma unroll
            for (int f = 0; f < 9; ++f) rec[f] = src[f];
          } else {  // tail records past the 16-B-multiple prefix
            const uint32_t *src = reinterpret_cast<const uint32_t *>(raw) + (sb + r) * 9;
#pragma unroll
            for (int f = 0; f < 9; ++f) rec[f] = __ldg(src + f);
          }
          sort_one(r, rec, (uint32_t)(r + 1) * sizeof(IdT) <= ib ? (int32_t)sid[r] : (int32_t)__ldg(ids + sb + r));
        }
      }
      __syncthreads();  // stage st fully read
      if (threadIdx.x == 0) issue(q + kTmaStages);
    }
    if (nbase < n) reserve_next();
    // 2) contiguous per-model runs out
    const int nk = (int)(end - base);
    for (int k = threadIdx.x; k < nk; k += kGBlock) {
      const uint32_t e = skey[k];
      const int m = (int)(e >> 16);
      const int32_t pos = basep[m] + (k - loff[m]);
      perm[pos] = (int32_t)(base + (e & 0xFFFFu));
      if (m < LAKE_MAX_MODELS) pdig[pos] = srow[k];
    }
    __syncthreads();
  }
}

__device__ __forceinline__ int find_model(const int32_t *off, int32_t t) {
  int lo = 0, hi = LAKE_MAX_MODELS;  // off[lo] <= t < off[hi]
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (off[mid] <= t) lo = mid; else hi = mid;
  }
  return lo;
}

// One thread per tile of either list (grid-stride), the model found by binary search over the
// per-model tile offsets staged in shared memory (searching them in global memory put ~10
// dependent L2 round trips in every thread: 10 us per call at C5).
__global__ void __launch_bounds__(256)
group_tiles(const WsHeader *__restrict__ h, int64_t max64, int64_t max256,
            int32_t *t64_model, int64_t *t64_begin, int32_t *t64_count,
            int32_t *t256_model, int64_t *t256_begin, int32_t *t256_count) {
  __shared__ int32_t off64[LAKE_MAX_MODELS + 1], off256[LAKE_MAX_MODELS + 1];
  __shared__ int32_t ord[LAKE_MAX_MODELS], cnt[LAKE_MAX_MODELS], offs[LAKE_MAX_MODELS];
  for (int i = threadIdx.x; i <= LAKE_MAX_MODELS; i += blockDim.x) {
    off64[i] = h->tile_off64[i];
    off256[i] = h->tile_off256[i];
    if (i < LAKE_MAX_MODELS) {
      ord[i] = h->ord256[i];
      cnt[i] = h->counts[i];
      offs[i] = h->offsets[i];
    }
  }
  __syncthreads();
  const int64_t n64 = h->n_tiles64 < max64 ? h->n_tiles64 : max64;
  const int64_t n256 = h->n_tiles256 < max256 ? h->n_tiles256 : max256;
  const int64_t nt = n64 > n256 ? n64 : n256;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < nt;
       t += (int64_t)gridDim.x * blockDim.x) {
    if (t < n64) {
      const int m = find_model(off64, (int32_t)t);
      const int32_t local = (int32_t)t - off64[m];
      const int32_t rem = cnt[m] - local * kF32TileM;
      t64_model[t] = m;
      t64_begin[t] = (int64_t)offs[m] + (int64_t)local * kF32TileM;
      t64_count[t] = rem < kF32TileM ? rem : kF32TileM;
    }
    if (t < n256) {
      const int k = find_model(off256, (int32_t)t);
      const int m = ord[k];
      const int32_t local = (int32_t)t - off256[k];
      const int32_t rem = cnt[m] - local * kTcTileRows;
      t256_model[t] = m;
      t256_begin[t] = (int64_t)offs[m] + (int64_t)local * kTcTileRows;
      t256_count[t] = rem < kTcTileRows ? rem : kTcTileRows;
    }
  }
}

__global__ void unknown_fill(const WsHeader *__restrict__ h, int64_t n,
                             const int32_t *__restrict__ perm, uint8_t *decisions,
                             float *logits) {
  const int64_t start = h->n_known;
  for (int64_t p = start + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x) {
    const int32_t io = perm[p];
    decisions[io] = 0;
    if (logits) {
      logits[(int64_t)io * 2] = __int_as_float(0x7fc00000);
      logits[(int64_t)io * 2 + 1] = __int_as_float(0x7fc00000);
    }
  }
}

}  // namespace

int64_t group_max_tiles(int64_t n, int tile_rows) {
  return (n + tile_rows - 1) / tile_rows + LAKE_MAX_MODELS;
}

size_t group_workspace_bytes(int64_t n) { return ws_layout(n).total; }

GroupView group_view(void *ws, int64_t n) {
  const WsLayout L = ws_layout(n);
  uint8_t *b = static_cast<uint8_t *>(ws);
  WsHeader *h = reinterpret_cast<WsHeader *>(b + L.header);
  GroupView v{};
  v.perm = reinterpret_cast<int32_t *>(b + L.perm);
  v.n_unknown = &h->n_unknown;
  v.counts = h->counts;
  return v;
}

struct GroupPtrs {
  WsHeader *h;
  int32_t *perm;
  int32_t *tm[2];
  int64_t *tb[2];
  int32_t *tc[2];
  int32_t *nt[2];
  int32_t *split;  // NN-class prefix of the 256-row tile list
  int64_t max[2];
  int32_t *cc;  // per-chunk histograms
  uint4 *pdig;  // packed digit rows, grouped order
  int32_t *cursor;  // padded per-model scatter cursors
};

static GroupPtrs group_ptrs(void *ws, int64_t n) {
  const WsLayout L = ws_layout(n);
  uint8_t *b = static_cast<uint8_t *>(ws);
  GroupPtrs p{};
  p.h = reinterpret_cast<WsHeader *>(b + L.header);
  p.perm = reinterpret_cast<int32_t *>(b + L.perm);
  p.tm[0] = reinterpret_cast<int32_t *>(b + L.t64_model);
  p.tb[0] = reinterpret_cast<int64_t *>(b + L.t64_begin);
  p.tc[0] = reinterpret_cast<int32_t *>(b + L.t64_count);
  p.tm[1] = reinterpret_cast<int32_t *>(b + L.t256_model);
  p.tb[1] = reinterpret_cast<int64_t *>(b + L.t256_begin);
  p.tc[1] = reinterpret_cast<int32_t *>(b + L.t256_count);
  p.cc = reinterpret_cast<int32_t *>(b + L.chunk_counts);
  p.pdig = reinterpret_cast<uint4 *>(b + L.pdig);
  p.cursor = reinterpret_cast<int32_t *>(b + L.cursor);
  p.nt[0] = &p.h->n_tiles64;
  p.nt[1] = &p.h->n_tiles256;
  p.split = &p.h->n_tiles256_nn;
  p.max[0] = L.max64;
  p.max[1] = L.max256;
  return p;
}

cudaError_t launch_group(int64_t n, const void *model_ids, int id_kind, const DevModel *table,
                         void *ws, const void *in, int in_kind, cudaStream_t s) {
  GroupPtrs p = group_ptrs(ws, n);
  group_init<<<1, LAKE_MAX_MODELS, 0, s>>>(table, p.h);
  int dev = 0;
  cudaGetDevice(&dev);
  static std::atomic<int> sms_cache[64];  // per-device SM count (a race repeats the query)
  int sms = sms_cache[dev & 63].load(std::memory_order_relaxed);
  if (!sms) {
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) sms = 148;
    sms_cache[dev & 63].store(sms, std::memory_order_relaxed);
  }
  const int64_t chunks = (n + kChunk - 1) / kChunk;
  // 4 blocks of 512 threads per SM: full occupancy (32 registers), enough loads in flight
  const int grid = (int)(chunks < 4 * sms ? chunks : 4 * sms);
  auto hist = [&](auto *ids) {
    if (grid > 0) group_hist<<<grid, kGBlock, 0, s>>>(ids, n, p.h, p.cc);
  };
  auto scatter_pack = [&](auto kern, auto *ids) {
    static std::atomic<bool> attr[64];  // per device; a race repeats the attribute call
    if (!attr[dev & 63].load(std::memory_order_acquire)) {
      cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kPackSmem);
      attr[dev & 63].store(true, std::memory_order_release);
    }
    const int pgrid = (int)(chunks < 2 * sms ? chunks : 2 * sms);
    kern<<<pgrid, kGBlock, kPackSmem, s>>>(ids, n, p.h, p.perm, p.cc, in, p.pdig, p.cursor);
  };
  auto scatter = [&](auto *ids) {
    using IdT = std::remove_cv_t<std::remove_pointer_t<decltype(ids)>>;
    if (grid <= 0) return;
    if (!in)
      group_scatter<IdT, -1><<<grid, kGBlock, 0, s>>>(ids, n, p.h, p.perm, p.cc, nullptr, nullptr,
                                                      p.cursor);
    else if (in_kind == LAKE_IN_RAW && LAKE_SCATTER_TMA &&
             (reinterpret_cast<uintptr_t>(in) & 15) == 0 && (reinterpret_cast<uintptr_t>(ids) & 15) == 0) {
      auto kern = group_scatter_pack_tma<IdT>;
      static std::atomic<bool> attr_t[64];
      if (!attr_t[dev & 63].load(std::memory_order_acquire)) {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTmaSmem);
        attr_t[dev & 63].store(true, std::memory_order_release);
      }
      const int tgrid = (int)(chunks < sms ? chunks : sms);
      kern<<<tgrid, kGBlock, kTmaSmem, s>>>(ids, n, p.h, p.perm, p.cc, in, p.pdig, p.cursor);
    } else if (in_kind == LAKE_IN_RAW)
      scatter_pack(group_scatter_pack<IdT, LAKE_IN_RAW>, ids);
    else
      scatter_pack(group_scatter_pack<IdT, LAKE_IN_DIGITS>, ids);
  };
  const int32_t *i32 = static_cast<const int32_t *>(model_ids);
  const uint16_t *u16 = static_cast<const uint16_t *>(model_ids);
  const uint8_t *u8 = static_cast<const uint8_t *>(model_ids);
  if (id_kind == 1) hist(u16); else if (id_kind == 2) hist(u8); else hist(i32);
  group_scan<<<1, LAKE_MAX_MODELS, 0, s>>>(p.h, p.cursor);
  if (id_kind == 1) scatter(u16); else if (id_kind == 2) scatter(u8); else scatter(i32);
  const int64_t mt = p.max[0] > p.max[1] ? p.max[0] : p.max[1];
  const int64_t tblocks = (mt + 255) / 256 < 2 * sms ? (mt + 255) / 256 : 2 * sms;
  group_tiles<<<(unsigned)(tblocks > 0 ? tblocks : 1), 256, 0, s>>>(p.h, p.max[0], p.max[1], p.tm[0],
                                                           p.tb[0], p.tc[0], p.tm[1], p.tb[1],
                                                           p.tc[1]);
  count_launch(grid > 0 ? 5 : 3);
  return cudaGetLastError();
}

// Fill a TileSched for the grouped launch; which = 0 (64-row FP32 tiles) / 1 (256-row TC).
cudaError_t launch_group_pack(void *ws, int64_t n, const void *in, int in_kind, cudaStream_t s) {
  GroupPtrs p = group_ptrs(ws, n);
  const int grid = (int)((n + 255) / 256 < 4 * 148 ? (n + 255) / 256 : 4 * 148);
  if (grid <= 0) return cudaSuccess;
  if (in_kind == LAKE_IN_RAW) group_pack<LAKE_IN_RAW><<<grid, 256, 0, s>>>(p.h, p.perm, in, p.pdig);
  else group_pack<LAKE_IN_DIGITS><<<grid, 256, 0, s>>>(p.h, p.perm, in, p.pdig);
  count_launch();
  return cudaGetLastError();
}

void group_sched(void *ws, int64_t n, int which, const DevModel *table, TileSched *ts) {
  GroupPtrs p = group_ptrs(ws, n);
  ts->tile_split_dev = which == 1 ? p.split : nullptr;
  ts->pdig = which == 1 ? p.pdig : nullptr;
  ts->tile_model = p.tm[which];
  ts->tile_begin = p.tb[which];
  ts->tile_count = p.tc[which];
  ts->perm = p.perm;
  ts->n_tiles_dev = p.nt[which];
  ts->n_tiles = p.max[which];
  ts->n = n;
  ts->table = table;
}

cudaError_t launch_unknown_fill(void *ws, int64_t n, uint8_t *decisions, float *logits,
                                cudaStream_t s) {
  GroupPtrs p = group_ptrs(ws, n);
  unknown_fill<<<64, 256, 0, s>>>(p.h, n, p.perm, decisions, logits);
  count_launch();
  return cudaGetLastError();
}

}  // namespace lake
