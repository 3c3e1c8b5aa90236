// mlp_tc2.cu — fused digitise -> MLP -> argmax on tcgen05 tensor cores, fp16 / bf16 operands,
// TWO 256-row tiles in flight per CTA pair (the default fp16/bf16 kernel; tf32 runs
// mlp_tc.cu, whose weights do not leave room for this kernel's SMEM H ring).
//
// Network: "two layers with 256 and 2 neurons" and the +1 / +2 variants with extra
// 256-wide hidden layers (§7.1); hidden ReLU, biases (R11, R12);
// decision = logit1 > logit0 (R14). Batch scoring = score_features (Table 1).
//
// Why two tiles: with one tile in flight, every layer's epilogue (TMEM ->
// bias/ReLU -> operand type) sits on the critical path between two MMA layers of the same
// tile, and the tensor pipe idles about half the time. Here a CTA pair keeps two tiles, A
// and B, each with ONE 256-column fp32 accumulator in TMEM (A: columns 0-255, B: 256-511),
// and two epilogue groups (group 0 serves tile A, group 1 tile B). The MMA thread alternates
// layers between the tiles — L0(A) L0(B) L1(A) L1(B) L2(A) L2(B) — so while the tensor
// cores run a layer of one tile, the other tile's epilogue drains its accumulator.
//
// H (the next layer's A operand) goes through ONE SMEM ring of 8 chunk slots (32 features x
// 128 rows, 8 KB each, 64 KB): the fills happen in the fixed order H0(A) H0(B) H1(A) H1(B)
// ... and the MMAs consume them in the same order, so a slot is refilled by the other tile's
// epilogue as soon as the MMA has read it (tcgen05.commit -> HFREE). One ring instead of two
// H tiles is what makes NN+2's 136 KB of fp16 weights, 64 KB of H and 16 KB of X fit in SMEM.
//
// Tiles are paired into "units" of two consecutive tiles of the same model (a tile whose
// model differs from its neighbour's forms a unit alone); weights are reloaded only between
// units.
//
// Warp roles (20 warps): w0-1 digitisers (raw records -> operand-type digits, X double
// buffer), w2 weight loader + TMEM allocator, w3-10 epilogue group 0 (tile A), w11-18
// epilogue group 1 (tile B), w19 MMA issuer (leader CTA, one thread). An epilogue warp owns
// TMEM lane quadrant (warp % 4) and the 32-column chunks hh, hh+2, hh+4, hh+6 (hh = which of
// the quadrant's two warps), i.e. 32 rows x 128 columns of its tile's accumulator.
//
// Synchronisation (mbarriers, CTA-scope acquire; leader CTA unless noted):
//   xfull/xempty[2]  digitisers <-> MMA            (X double buffer; xempty in both CTAs)
//   dfull[2]         MMA commit -> epilogue group s (accumulator s holds a finished layer)
//   tempty[2]        epilogue group s -> MMA        (accumulator s drained)
//   hfull[8]         epilogue warps -> MMA          (ring slot written: 4 warps x 2 CTAs)
//   hfree[8]         MMA commit -> epilogue warps   (ring slot read; both CTAs)
//   wload/wready/wfree  weights (as in mlp_tc.cu)
// A producer of ring fill f waits for consumption f-1 only when consumption f-2 is already
// complete (its own layer's dfull implies it), so mbarrier parity never aliases.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <atomic>

#include "digitize.cuh"
#include "lake_internal.h"
#include "lake_ptx.cuh"

// ---- optional timeline trace (make trace): clock64 stamps of the leader CTA of cluster 0;
// streams: 0 MMA thread, 1 epilogue warp 3 (quadrant 3, chunks 0/4), 2 epilogue warp 18,
// 3 digitiser thread 0; 2 u64 per event, 64K events per stream
#ifdef LAKE_TRACE
__device__ unsigned long long *g_lake_trace2 = nullptr;
#define LAKE_TEV2(kind, tile, layer, x)                                                     \
  do {                                                                                   \
    if (tr_stream >= 0 && tr_i < (1u << 16)) {                                           \
      unsigned long long *p_ = tr_buf + 2ull * (tr_stream * (1u << 16) + tr_i++);         \
      p_[0] = ((unsigned long long)(kind) << 56) | ((unsigned long long)(tile) << 24) |    \
              ((unsigned long long)(layer) << 8) | (unsigned long long)(x);              \
      p_[1] = clock64();                                                                 \
    }                                                                                    \
  } while (0)
#else
#define LAKE_TEV2(kind, tile, layer, x) do {} while (0)
#endif

namespace lake {
namespace {

constexpr int kThreads2 = 32 * 20;
constexpr uint32_t kWarpDig = 0, kWarpLoad = 2, kWarpEpi = 3, kWarpMma = 19;
constexpr uint32_t kEpiWarps = 16;
constexpr uint32_t kRingSlots = 8;                      // = H chunks per layer
constexpr uint32_t kChunkCols = kHidden / kRingSlots;   // 32 features per chunk / slot
constexpr uint32_t kSlotBytes = 128 * kChunkCols * 2;   // 8 KB
constexpr uint32_t kXBytes = 128 * kTcK0 * 2;           // 8 KB
constexpr uint32_t kLbo = 128 * 16;                     // K-direction core stride (128 rows)
constexpr uint32_t kPrmFloats = kHidden + 2 * kHidden + 4;  // last bias | W_out | b_out
constexpr uint32_t kHBiasFloats = (kMaxHiddenLayers - 1) * kHidden;
constexpr uint32_t kRedBytes = 3 * 128 * 2 * 4;         // partial logits of 3 warps/quadrant

__host__ __device__ constexpr uint32_t al1k(uint32_t x) { return (x + 1023u) & ~1023u; }

struct Layout2 {
  uint32_t ring, x, prm, hbias, red, bar, total;
};
__host__ __device__ constexpr Layout2 tc2_layout(int nh_layout) {
  Layout2 L{};
  L.ring = al1k(tc_image_bytes(nh_layout, 0));
  L.x = L.ring + (nh_layout > 1 ? kRingSlots * kSlotBytes : 0u);
  L.prm = L.x + 2 * kXBytes;
  L.hbias = L.prm + kPrmFloats * 4;
  L.red = L.hbias + kHBiasFloats * 4;
  L.bar = L.red + kRedBytes;
  L.total = L.bar + 256;
  return L;
}
static_assert(tc2_layout(3).total <= 232448, "NN+2 two-tile layout exceeds 227 KB");

enum : uint32_t {
  B_WLOAD = 0, B_WREADY = 1, B_WFREE = 2, B_XFULL = 3, B_XEMPTY = 5, B_DFULL = 7,
  B_TEMPTY = 9, B_HFULL = 11, B_HFREE = B_HFULL + kRingSlots, B_COUNT = B_HFREE + kRingSlots
};
constexpr uint32_t kTmemSlot = B_COUNT * 8;
static_assert(kTmemSlot + 4 <= 256, "barrier block");

struct TileInfo {
  const DevModel *model;
  const uint8_t *img;
  int64_t begin;
  int count;
  int nh;
};

template <int PREC>
__device__ __forceinline__ TileInfo tile_info(const TileSched &ts, int64_t t) {
  TileInfo ti;
  if (ts.tile_model) {
    ti.model = &ts.table[ts.tile_model[t]];
    ti.begin = ts.tile_begin[t];
    ti.count = ts.tile_count[t];
  } else {
    ti.model = &ts.model;
    ti.begin = t * kTcTileRows;
    const int64_t rem = ts.n - ti.begin;
    ti.count = (int)(rem < kTcTileRows ? rem : kTcTileRows);
  }
  ti.img = ti.model->tc_img[PREC];
  ti.nh = ti.model->nh;
  return ti;
}

// A unit: tile t alone, or tiles t and t+1 when both belong to the same model. Every role
// walks the same unit sequence.
template <int PREC>
__device__ __forceinline__ int unit_at(const TileSched &ts, int64_t t, int64_t t_end,
                                       TileInfo &a, TileInfo &b) {
  a = tile_info<PREC>(ts, t);
  if (t + 1 < t_end) {
    b = tile_info<PREC>(ts, t + 1);
    if (b.img == a.img) return 2;
  }
  return 1;
}

// Last hidden layer: ReLU(acc + b) in fp32, accumulated straight into the two logits.
__device__ __forceinline__ void epi_logits32(const uint32_t (&r)[32], const float *bl,
                                             const float *wo, uint32_t col0, float (&p)[4]) {
#pragma unroll
  for (int c4 = 0; c4 < 8; ++c4) {
    const float4 b4 = *reinterpret_cast<const float4 *>(bl + col0 + c4 * 4);
    const float4 w0 = *reinterpret_cast<const float4 *>(wo + col0 + c4 * 4);
    const float4 w1 = *reinterpret_cast<const float4 *>(wo + kHidden + col0 + c4 * 4);
    const float bb[4] = {b4.x, b4.y, b4.z, b4.w};
    const float ww0[4] = {w0.x, w0.y, w0.z, w0.w};
    const float ww1[4] = {w1.x, w1.y, w1.z, w1.w};
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      float h = __uint_as_float(r[c4 * 4 + e]) + bb[e];
      h = h > 0.0f ? h : 0.0f;
      p[(e & 1) * 2 + 0] = fmaf(h, ww0[e], p[(e & 1) * 2 + 0]);
      p[(e & 1) * 2 + 1] = fmaf(h, ww1[e], p[(e & 1) * 2 + 1]);
    }
  }
}

// Hidden layer chunk: 32 fp32 accumulator columns of one row -> + bias (fp32) -> ReLU and one
// rounding to the operand type -> 16 packed words (the row's 64 bytes of this ring slot).
template <int PREC>
__device__ __forceinline__ void epi_h32(const uint32_t (&r)[32], const float *bias,
                                        uint32_t (&w)[16]) {
#pragma unroll
  for (int c4 = 0; c4 < 8; ++c4) {
    const float4 b4 = *reinterpret_cast<const float4 *>(bias + c4 * 4);
    const float v0 = __uint_as_float(r[c4 * 4 + 0]) + b4.x;
    const float v1 = __uint_as_float(r[c4 * 4 + 1]) + b4.y;
    const float v2 = __uint_as_float(r[c4 * 4 + 2]) + b4.z;
    const float v3 = __uint_as_float(r[c4 * 4 + 3]) + b4.w;
    if constexpr (PREC == 0) {
      w[c4 * 2 + 0] = ptx::relu_pack_f16(v0, v1);
      w[c4 * 2 + 1] = ptx::relu_pack_f16(v2, v3);
    } else {
      w[c4 * 2 + 0] = ptx::relu_pack_bf16(v0, v1);
      w[c4 * 2 + 1] = ptx::relu_pack_bf16(v2, v3);
    }
  }
}

template <int PREC, int IN_KIND>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads2, 1)
mlp_tc2_kernel(const void *__restrict__ in, const __grid_constant__ TileSched ts, int nh_layout,
               uint8_t *__restrict__ decisions, float *__restrict__ logits) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const Layout2 L = tc2_layout(nh_layout);
  const uint32_t sbase = ptx::smem_u32(smem);
  const uint32_t bar0 = sbase + L.bar;
  auto bar = [&](uint32_t slot) { return bar0 + slot * 8; };
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ptx::cluster_ctarank();
  const uint32_t cid = ptx::cluster_id_x(), ncl = ptx::num_clusters_x();
#ifdef LAKE_TRACE
  unsigned long long *const tr_buf = g_lake_trace2;
  const int tr_stream = !(tr_buf && cid == 0 && rank == 0) ? -1
                      : (warp == kWarpMma && lane == 0) ? 0 : (warp == kWarpEpi && lane == 0) ? 1
                      : (warp == kWarpEpi + kEpiWarps - 1 && lane == 0) ? 2
                      : (threadIdx.x == 0) ? 3 : -1;
  uint32_t tr_i = 0;
#endif
  const int64_t n_tiles = ts.n_tiles_dev ? (int64_t)*ts.n_tiles_dev : ts.n_tiles;
  const int64_t t_begin = n_tiles * cid / ncl;
  const int64_t t_end = n_tiles * (cid + 1) / ncl;

  if (threadIdx.x == 0) {
    ptx::mbar_init(bar(B_WLOAD), 1);
    ptx::mbar_init(bar(B_WREADY), 2);              // one arrive per CTA loader
    ptx::mbar_init(bar(B_WFREE), 1);               // tcgen05.commit (multicast)
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(bar(B_XFULL + i), 2);         // one arrive per CTA digitiser group
      ptx::mbar_init(bar(B_XEMPTY + i), 1);        // tcgen05.commit (multicast)
      ptx::mbar_init(bar(B_DFULL + i), 1);         // tcgen05.commit (multicast)
      ptx::mbar_init(bar(B_TEMPTY + i), 2 * kEpiWarps);   // every epilogue warp, both CTAs
    }
    for (uint32_t i = 0; i < kRingSlots; ++i) {
      ptx::mbar_init(bar(B_HFULL + i), 2 * 4);     // the chunk's 4 warps (one per quadrant), both CTAs
      ptx::mbar_init(bar(B_HFREE + i), 1);         // tcgen05.commit (multicast)
    }
    ptx::fence_mbar_init();
  }
  if (warp == kWarpLoad) {
    ptx::tmem_alloc_cg2(sbase + L.bar + kTmemSlot, 512);
    ptx::tmem_relinquish_cg2();
  }
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + L.bar + kTmemSlot);

  if (warp == kWarpLoad) {
    // ================= weight loader (both CTAs): the model's image at unit switches ====
    if (lane == 0) {
      const uint8_t *cur = nullptr;
      uint32_t wl_phase = 0, wf_phase = 0;
      const uint32_t wready_leader = ptx::mapa(bar(B_WREADY), 0);
      TileInfo a, b;
      for (int64_t t = t_begin; t < t_end;) {
        const int nt = unit_at<PREC>(ts, t, t_end, a, b);
        t += nt;
        if (a.img == cur) continue;
        if (cur) {  // every MMA reading the old weights has completed
          ptx::mbar_wait(bar(B_WFREE), wf_phase);
          wf_phase ^= 1;
        }
        const uint32_t bytes = tc_image_bytes(a.nh, PREC);
        const uint8_t *src = a.img + (size_t)rank * bytes;
        ptx::mbar_arrive_expect_tx(bar(B_WLOAD), bytes);
        for (uint32_t off = 0; off < bytes; off += 32768) {
          const uint32_t len = (bytes - off) < 32768 ? (bytes - off) : 32768;
          ptx::bulk_g2s(sbase + off, src + off, len, bar(B_WLOAD));
        }
        ptx::mbar_wait(bar(B_WLOAD), wl_phase);
        wl_phase ^= 1;
        ptx::mbar_arrive_cluster(wready_leader);
        cur = a.img;
      }
    }
  } else if (warp == kWarpMma) {
    // ================= MMA issuer (leader CTA) =================
    // The whole warp runs the schedule (waits, descriptor arithmetic) in converged,
    // warp-uniform code, so the operands live in uniform registers; only the tcgen05.mma /
    // commit issue is predicated on lane 0. (A lane-0-only region made the compiler wrap every
    // MMA in an ELECT / R2UR.BROADCAST / BRA.U.ANY loop and the issue thread, not the tensor
    // pipe, became the bound: ncu showed it in fixed-latency waits on those instructions.)
    if (rank == 0) {
      const bool issuer = lane == 0;
      const uint32_t tm = __shfl_sync(0xffffffffu, tmem, 0);  // provably warp-uniform
      const uint32_t idesc = ptx::umma_idesc_f16(PREC, 256, 256);
      constexpr uint64_t kStep = (2 * kLbo) >> 4;  // one K-step (16) = 2 core matrices
      const uint64_t xdesc0 = ptx::umma_desc(sbase + L.x, kLbo, 128);
      const uint64_t xdesc1 = ptx::umma_desc(sbase + L.x + kXBytes, kLbo, 128);
      const uint64_t w0desc = ptx::umma_desc(sbase, kLbo, 128);
      const uint64_t ringdesc = ptx::umma_desc(sbase + L.ring, kLbo, 128);
      const uint64_t wh1 = ptx::umma_desc(sbase + kTcW0HalfBytes, kLbo, 128);
      const uint64_t wh2 = ptx::umma_desc(sbase + kTcW0HalfBytes + kTcWhHalfBytes, kLbo, 128);
      constexpr uint64_t kSlotStep = kSlotBytes >> 4;
      const uint8_t *cur = nullptr;
      uint32_t w_phase = 0, t_phase = 0, used = 0, c = 0;  // c: ring fills consumed
      int64_t it = 0;                                        // tiles started (X buffers)
      auto acquire = [&](uint32_t s) {  // accumulator s drained by its epilogue group
        if (used & (1u << s)) {
          ptx::mbar_wait(bar(B_TEMPTY + s), (t_phase >> s) & 1);
          t_phase ^= (1u << s);
        }
        used |= (1u << s);
      };
      TileInfo a, b;
      for (int64_t t = t_begin; t < t_end;) {
        const int nt = unit_at<PREC>(ts, t, t_end, a, b);
        t += nt;
        if (a.img != cur) {
          ptx::mbar_wait(bar(B_WREADY), w_phase);
          w_phase ^= 1;
          cur = a.img;
        }
        const int nh = a.nh;
        for (int s = 0; s < nt; ++s, ++it) {  // layer 0: D = X[128(x2) x 32] * W0^T
          acquire(s);
          LAKE_TEV2(1, it, 0, s);  // tempty ok
          const uint32_t xb = (uint32_t)(it & 1);
          ptx::mbar_wait(bar(B_XFULL + xb), (uint32_t)((it >> 1) & 1));
          LAKE_TEV2(2, it, 0, s);  // xfull ok
          ptx::tc_fence_after();
          const uint32_t d = tm + s * 256;
          const uint64_t xd = xb ? xdesc1 : xdesc0;
#pragma unroll
          for (uint32_t k = 0; k < kTcK0 / 16; ++k)
            if (issuer) ptx::mma_f16_cg2(d, xd + k * kStep, w0desc + k * kStep, idesc, k);
          if (issuer) ptx::mma_commit_cg2(bar(B_XEMPTY + xb), 0x3);
          if (issuer) ptx::mma_commit_cg2(bar(B_DFULL + s), 0x3);
          __syncwarp();
        }
        for (int l = 1; l < nh; ++l) {  // hidden layers: A = H(l-1) from the ring
          const uint64_t wd = l == 1 ? wh1 : wh2;
          for (int s = 0; s < nt; ++s, ++c) {
            acquire(s);
            LAKE_TEV2(1, it, l, s);  // tempty ok
            ptx::tc_fence_after();
            const uint32_t d = tm + s * 256;
            for (uint32_t kc = 0; kc < kRingSlots; ++kc) {
              ptx::mbar_wait(bar(B_HFULL + kc), c & 1);
              LAKE_TEV2(3, it, l, s * 16 + kc);  // hfull ok
              ptx::tc_fence_after();
#pragma unroll
              for (uint32_t k = 0; k < kChunkCols / 16; ++k) {
                const uint32_t ks = kc * (kChunkCols / 16) + k;
                if (issuer)
                  ptx::mma_f16_cg2(d, ringdesc + kc * kSlotStep + k * kStep, wd + ks * kStep,
                                   idesc, ks);
              }
              if (issuer) ptx::mma_commit_cg2(bar(B_HFREE + kc), 0x3);
              __syncwarp();
            }
            if (issuer) ptx::mma_commit_cg2(bar(B_DFULL + s), 0x3);
            __syncwarp();
          }
        }
        if (t < t_end && tile_info<PREC>(ts, t).img != cur && issuer)
          ptx::mma_commit_cg2(bar(B_WFREE), 0x3);  // old weights no longer read
        __syncwarp();
      }
    }
  } else if (warp >= kWarpDig && warp < kWarpDig + 2) {
    // ================= digitisers: raw -> X (operand-type digits), 2 rows per thread ======
    // Software-pipelined one tile ahead: the dependent loads of tile t+1 (schedule entry ->
    // perm -> the records) are issued before tile t waits for its X buffer and is digitised,
    // so their latency overlaps tile t's work (with two tiles in flight the MMA consumes X
    // tiles twice as fast as one tile's layer chain did).
    const uint32_t d = threadIdx.x - kWarpDig * 32;  // 0..63
    const uint32_t xfull_leader0 = ptx::mapa(bar(B_XFULL), 0);
    auto gather = [&](int64_t t, uint32_t (&rec)[2][9], uint32_t &valid) {
      const TileInfo ti = tile_info<PREC>(ts, t);
      valid = 0;
#pragma unroll
      for (int half = 0; half < 2; ++half) {
        const int pos = (int)(rank * 128 + d + 64 * half);
        const bool v = pos < ti.count;
        valid |= (v ? 1u : 0u) << half;
        const int64_t p = ti.begin + (v ? pos : 0);
        const int64_t io = ts.perm ? (int64_t)ts.perm[p] : p;
        if (IN_KIND == LAKE_IN_RAW) {
          const uint32_t *src = reinterpret_cast<const uint32_t *>(in) + io * 9;
#pragma unroll
          for (int f = 0; f < 9; ++f) rec[half][f] = v ? __ldg(src + f) : 0u;
        } else {
          const uint4 *src = reinterpret_cast<const uint4 *>(
              reinterpret_cast<const uint8_t *>(in) + io * 32);
          uint4 v0 = make_uint4(0, 0, 0, 0), v1 = v0;
          if (v) {
            v0 = __ldg(src);
            v1 = __ldg(src + 1);
          }
          rec[half][0] = v0.x; rec[half][1] = v0.y; rec[half][2] = v0.z; rec[half][3] = v0.w;
          rec[half][4] = v1.x; rec[half][5] = v1.y; rec[half][6] = v1.z; rec[half][7] = v1.w;
          rec[half][8] = 0;
        }
      }
    };
    uint32_t cur[2][9], nxt[2][9], cvalid = 0, nvalid = 0;
    if (t_begin < t_end) gather(t_begin, cur, cvalid);
    int64_t it = 0;
    for (int64_t t = t_begin; t < t_end; ++t, ++it) {
      if (t + 1 < t_end) gather(t + 1, nxt, nvalid);
      const uint32_t xb = (uint32_t)(it & 1);
      LAKE_TEV2(8, it, 0, 0);  // gathered next
      ptx::mbar_wait(bar(B_XEMPTY + xb), (uint32_t)(((it >> 1) & 1) ^ 1));
      LAKE_TEV2(9, it, 0, 0);  // xempty ok
      const uint32_t xs = sbase + L.x + xb * kXBytes;
#pragma unroll
      for (int half = 0; half < 2; ++half) {
        const uint32_t r = d + 64 * half;
        uint32_t dg[32];
#pragma unroll
        for (int i = 0; i < 32; ++i) dg[i] = 0;
        if (cvalid & (1u << half)) {
          if (IN_KIND == LAKE_IN_RAW) {
            digitize_record(cur[half], [&](int k, uint32_t v) { dg[k] = v; });
          } else {
#pragma unroll
            for (int k = 0; k < 31; ++k) dg[k] = (cur[half][k >> 2] >> ((k & 3) * 8)) & 0xFFu;
          }
        }
        // value pairs by packed arithmetic: the 16-bit pattern M | v is the value M' + v
        // (fp16: 0x6400 = 1024, ulp 1 on [1024, 2048); bf16: 0x4300 = 128, ulp 1 on [128,
        // 256)), so one packed subtract of (M', M') yields (v0, v1) exactly (v < 128 for
        // bf16: digit bytes of LAKE_IN_DIGITS input convert value by value there)
        uint32_t w[16];
        constexpr uint32_t kMagic2 = PREC == 0 ? 0x64006400u : 0x43004300u;
#pragma unroll
        for (int pp = 0; pp < 16; ++pp) {
          if (IN_KIND == LAKE_IN_RAW || PREC == 0) {
            const uint32_t u = dg[2 * pp] | (dg[2 * pp + 1] << 16) | kMagic2;
            w[pp] = PREC == 0 ? ptx::sub_f16x2(u, kMagic2) : ptx::sub_bf16x2(u, kMagic2);
          } else {
            w[pp] = (uint32_t)__bfloat16_as_ushort(__uint2bfloat16_rn(dg[2 * pp])) |
                    ((uint32_t)__bfloat16_as_ushort(__uint2bfloat16_rn(dg[2 * pp + 1])) << 16);
          }
        }
#pragma unroll
        for (int kg = 0; kg < 4; ++kg)
          ptx::st_shared_v4(xs + kg * kLbo + r * 16, w[kg * 4 + 0], w[kg * 4 + 1],
                            w[kg * 4 + 2], w[kg * 4 + 3]);
      }
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(1, 64);
      if (d == 0) ptx::mbar_arrive_cluster(xfull_leader0 + xb * 8);
      LAKE_TEV2(10, it, 0, 0);  // x arrived
#pragma unroll
      for (int half = 0; half < 2; ++half)
#pragma unroll
        for (int f = 0; f < 9; ++f) cur[half][f] = nxt[half][f];
      cvalid = nvalid;
    }
  } else if (warp >= kWarpEpi && warp < kWarpEpi + kEpiWarps) {
    // ================= epilogue (16 warps, serve both tiles in MMA order) =================
    // Per layer and tile a warp loads its two 32-column chunks (hh, hh+4) of its quadrant's
    // rows, converts them in registers and only then signals the accumulator drained (so the
    // MMA may overwrite it with the tile's next layer at once); the converted H chunks are
    // then written into the ring as the MMA frees their slots.
    const uint32_t lw = warp - kWarpEpi;
    const uint32_t q = warp & 3;                           // TMEM lane quadrant
    const uint32_t hh = lw >> 2;                           // chunks hh and hh + 4
    const uint32_t row = q * 32 + lane;                    // row within this CTA's 128
    const uint32_t et = lw * 32 + lane;                    // 0..511
    const uint32_t hfull_leader0 = ptx::mapa(bar(B_HFULL), 0);
    const uint32_t tempty_leader0 = ptx::mapa(bar(B_TEMPTY), 0);
    float *prm = reinterpret_cast<float *>(smem + L.prm);    // last b | W_out | b_out
    float *hbias = reinterpret_cast<float *>(smem + L.hbias);
    float *red = reinterpret_cast<float *>(smem + L.red);     // [3][128][2] partial logits
    const uint32_t red_bar = 4 + q;                       // named barrier of the quadrant
    const uint32_t ring_row = sbase + L.ring + row * 16;
    const float *wo = prm + kHidden;
    const DevModel *cur = nullptr;
    uint32_t d_phase = 0, f = 0;  // d_phase: bit per tile slot; f: ring fills before the unit
    TileInfo a, b;
    for (int64_t t = t_begin; t < t_end;) {
      const int nt = unit_at<PREC>(ts, t, t_end, a, b);
      t += nt;
      const int nh = a.nh;
      if (a.model != cur) {
        // stage the model's epilogue parameters: fp32 biases of the H layers, fp32
        // last-layer bias | W_out | b_out
        ptx::named_bar_sync(2, kEpiWarps * 32);
        for (uint32_t i = et; i < (uint32_t)(nh - 1) * kHidden / 4; i += kEpiWarps * 32)
          reinterpret_cast<float4 *>(hbias)[i] =
              __ldg(reinterpret_cast<const float4 *>(a.model->b[0]) + i);
        const float4 *src = reinterpret_cast<const float4 *>(a.model->b[nh - 1]);
        for (uint32_t i = et; i < kPrmFloats / 4; i += kEpiWarps * 32)
          reinterpret_cast<float4 *>(prm)[i] = __ldg(src + i);
        ptx::named_bar_sync(2, kEpiWarps * 32);
        cur = a.model;
      }
      for (int l = 0; l < nh; ++l) {
        for (int s = 0; s < nt; ++s) {
          const TileInfo &ti = s == 0 ? a : b;
          ptx::mbar_wait(bar(B_DFULL + s), (d_phase >> s) & 1);
          d_phase ^= 1u << s;
          LAKE_TEV2(4, t, l, s);  // dfull ok
          ptx::tc_fence_after();
          const uint32_t tbase = tmem + ((q * 32) << 16) + s * 256;
          const uint32_t c0 = hh, c1 = hh + 4;
          uint32_t ra[32], rb[32];
#ifdef LAKE_ABL_EPI_NOP  // timing-only ablation: no accumulator reads
#pragma unroll
          for (int i = 0; i < 32; ++i) { ra[i] = i; rb[i] = tbase + i; }
#else
          ptx::tmem_ld_32x32b_x32(tbase + c0 * kChunkCols, ra);
          ptx::tmem_ld_32x32b_x32(tbase + c1 * kChunkCols, rb);
          ptx::tmem_ld_wait();
#endif
          if (l + 1 < nh) {
            // hidden layer -> H(l) of tile s into the ring (fill index fi)
            const uint32_t fi = f + (uint32_t)(l * nt + s);
            const float *bias = hbias + l * kHidden;
            uint32_t w0[16], w1[16];
            epi_h32<PREC>(ra, bias + c0 * kChunkCols, w0);
            epi_h32<PREC>(rb, bias + c1 * kChunkCols, w1);
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive_cluster(tempty_leader0 + s * 8);  // acc read
            LAKE_TEV2(5, t, l, s);  // converted, tempty arrived
#pragma unroll
            for (int j = 0; j < 2; ++j) {
              const uint32_t kc = j ? c1 : c0;
              const uint32_t(&w)[16] = j ? w1 : w0;
              if (fi > 0) ptx::mbar_wait(bar(B_HFREE + kc), (fi - 1) & 1);
              LAKE_TEV2(6, t, l, s * 16 + kc);  // hfree ok
              const uint32_t dst = ring_row + kc * kSlotBytes;
#ifdef LAKE_ABL_EPI_NOP  // timing-only ablation: no ring stores / proxy fence
              if (w[0] == 0x12345678u && w[5] == 0x9abcdef0u)
#endif
              {
#pragma unroll
                for (int kg = 0; kg < 4; ++kg)
                  ptx::st_shared_v4(dst + kg * kLbo, w[kg * 4 + 0], w[kg * 4 + 1], w[kg * 4 + 2],
                                    w[kg * 4 + 3]);
                ptx::fence_proxy_async_smem();
              }
              __syncwarp();
              if (lane == 0) ptx::mbar_arrive_cluster(hfull_leader0 + kc * 8);
            }
          } else {
            // last hidden layer: fold the 2-neuron output layer (fp32, CUDA cores)
            float p[4] = {0.0f, 0.0f, 0.0f, 0.0f};
            epi_logits32(ra, prm, wo, c0 * kChunkCols, p);
            epi_logits32(rb, prm, wo, c1 * kChunkCols, p);
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive_cluster(tempty_leader0 + s * 8);  // acc read
            float p0 = p[0] + p[2], p1 = p[1] + p[3];
            // combine the quadrant's 4 warps: slices 1..3 write partials, slice 0 sums
            if (hh > 0) {
              red[((hh - 1) * 128 + row) * 2 + 0] = p0;
              red[((hh - 1) * 128 + row) * 2 + 1] = p1;
            }
            ptx::named_bar_sync(red_bar, 128);
            if (hh == 0) {
#pragma unroll
              for (int j = 0; j < 3; ++j) {
                p0 += red[(j * 128 + row) * 2 + 0];
                p1 += red[(j * 128 + row) * 2 + 1];
              }
              const float l0 = p0 + wo[2 * kHidden + 0];
              const float l1 = p1 + wo[2 * kHidden + 1];
              const int pos = (int)(rank * 128 + row);
              if (pos < ti.count) {
                const int64_t pp = ti.begin + pos;
                const int64_t io = ts.perm ? (int64_t)ts.perm[pp] : pp;
                if (logits) {
                  logits[io * 2 + 0] = l0;
                  logits[io * 2 + 1] = l1;
                }
                decisions[io] = (l1 > l0) ? 1 : 0;
              }
            }
            ptx::named_bar_sync(red_bar, 128);  // partials read before they are rewritten
            LAKE_TEV2(7, t, l, s);  // logits done
          }
        }
      }
      f += (uint32_t)((nh - 1) * nt);
    }
  }

  __syncwarp();  // reconverge role lanes before the .aligned cluster barrier
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == kWarpLoad) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_cg2(tmem, 512);
  }
}

template <int PREC, int IN_KIND>
cudaError_t launch2_t(const void *in, const TileSched &ts, int nh_layout, uint8_t *dec,
                      float *logits, cudaStream_t s, int grid) {
  const Layout2 L = tc2_layout(nh_layout);
  static std::atomic<bool> attr_set[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (!attr_set[dev & 63].load(std::memory_order_acquire)) {
    cudaError_t e = cudaFuncSetAttribute(mlp_tc2_kernel<PREC, IN_KIND>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)tc2_layout(kMaxHiddenLayers).total);
    if (e != cudaSuccess) return e;
    attr_set[dev & 63].store(true, std::memory_order_release);
  }
  mlp_tc2_kernel<PREC, IN_KIND><<<grid, kThreads2, L.total, s>>>(in, ts, nh_layout, dec, logits);
  return cudaGetLastError();
}

}  // namespace

#ifdef LAKE_TRACE
extern "C" int lake_trace2_set(void *dev_buf) {
  return (int)cudaMemcpyToSymbol(g_lake_trace2, &dev_buf, sizeof(void *));
}
#endif

cudaError_t launch_mlp_tc2(const void *in, int in_kind, int prec, const TileSched &ts, int nh,
                           int grid, uint8_t *decisions, float *logits, cudaStream_t s) {
  if (prec == 0)
    return in_kind == LAKE_IN_RAW ? launch2_t<0, LAKE_IN_RAW>(in, ts, nh, decisions, logits, s, grid)
                                  : launch2_t<0, LAKE_IN_DIGITS>(in, ts, nh, decisions, logits, s, grid);
  return in_kind == LAKE_IN_RAW ? launch2_t<1, LAKE_IN_RAW>(in, ts, nh, decisions, logits, s, grid)
                                : launch2_t<1, LAKE_IN_DIGITS>(in, ts, nh, decisions, logits, s, grid);
}

}  // namespace lake
