// mlp_tc.cu — fused digitise -> MLP -> argmax on the 5th-generation tensor cores
// (tcgen05, sm_100a), fp16 or bf16 operands, fp32 accumulation in TMEM.
//
// Network: "two layers with 256 and 2 neurons" and the +1 / +2 variants with extra
// 256-wide hidden layers (§7.1); hidden ReLU, biases (R11, R12);
// decision = logit1 > logit0 (R14). Batch scoring = score_features (Table 1).
//
// Design:
//  * A cluster of 2 CTAs (one CTA pair, cta_group::2) owns 256-row tiles. Each CTA holds
//    128 rows of the activations (A operand, SMEM) and of every accumulator (TMEM lanes),
//    and HALF of every 256-wide weight matrix (B operand, N/2 rows), resident in SMEM for
//    the whole launch: NN+2's W0..W2 are 272 KB in fp16, 136 KB per CTA.
//  * Hidden layers run on the tensor cores: X[128x32] -> L0 (K=32) -> H[128x256] -> L1..
//    (K=256). The 2-wide output layer is folded into the last hidden layer's epilogue on
//    CUDA cores (fp32), so no N=2->16 padded MMA and no extra TMEM round trip per tile.
//  * Accumulators alternate between two 256-column TMEM buffers (all 512 columns): while
//    the MMA of layer l+1 runs into one, the epilogue drains layer l from the other. The
//    epilogue writes H in 64-column chunks and signals each, so layer l+1's MMA starts on
//    K-chunk 0 while later chunks are still being converted.
//  * Warp roles (12 warps): w0 weight loader + TMEM allocator, w1 MMA issuer (leader CTA,
//    one thread), w2-3 digitisers (raw records -> fp16 digits, double-buffered X),
//    w4-11 epilogue (tcgen05.ld -> +bias -> ReLU -> fp16 -> st.shared -> mbarrier; the last
//    layer: -> W_out dot products -> logits / decision). Biases and W_out (fp32) are staged
//    into SMEM by the epilogue warps themselves whenever the tile's model changes.
//  * Operand layout: K-major, SWIZZLE_NONE core matrices (8 rows x 16 B), core (rg, kg) at
//    kg * R*16 + rg*128: the epilogue's per-row 16-byte stores from 32 consecutive rows
//    are 512 contiguous bytes (bank-conflict free).
//  * Synchronisation (all mbarriers, CTA-scope acquire; see lake_ptx.cuh):
//      xfull/xempty[2]  digitisers <-> MMA              (X double buffer)
//      dfull[2]         MMA commit -> epilogues         (accumulator b ready)
//      tempty[2]        epilogues (16 warps) -> MMA     (accumulator b drained)
//      hready[4]        epilogues (16 warps) -> MMA     (H K-chunk written)
//      wload/wready     loaders -> MMA                  (weights resident)
//      wfree            MMA commit -> loaders           (old model's last MMA done)
//    Every producer/consumer pair is kept within one phase of each other by a reverse
//    dependency, so mbarrier parity never aliases.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "digitize.cuh"
#include "lake_internal.h"
#include "lake_ptx.cuh"

namespace lake {
namespace {

constexpr int kThreads = 384;
constexpr uint32_t kHBytes = 128 * kHidden * 2;   // 64 KB
constexpr uint32_t kXBytes = 128 * kTcK0 * 2;     // 8 KB
constexpr uint32_t kLboR128 = 128 * 16;           // K-direction core stride, 128-row operand
constexpr uint32_t kPrmFloats = kMaxHiddenLayers * kHidden + 2 * kHidden + 4;  // biases|Wout|bout
constexpr uint32_t kRedBytes = 2 * 128 * 2 * 4;   // output-layer half sums, double-buffered

__host__ __device__ constexpr uint32_t align1k(uint32_t x) { return (x + 1023u) & ~1023u; }

struct Layout {
  uint32_t h, x, prm, red, bar, total;
};
__host__ __device__ constexpr Layout tc_layout(int nh_layout) {
  Layout L{};
  L.h = align1k(tc_image_bytes(nh_layout));
  L.x = L.h + kHBytes;
  L.prm = L.x + 2 * kXBytes;
  L.red = L.prm + kPrmFloats * 4;
  L.bar = L.red + kRedBytes;
  L.total = L.bar + 256;
  return L;
}

// barrier slots (8 bytes each) inside the barrier block
enum : uint32_t {
  B_WLOAD = 0, B_WREADY = 1, B_XFULL = 2, B_XEMPTY = 4, B_DFULL = 6, B_TEMPTY = 8,
  B_HREADY = 10, B_WFREE = 14, B_COUNT = 15
};
constexpr uint32_t kTmemSlot = B_COUNT * 8;  // u32 TMEM base address

struct TileInfo {
  const DevModel *model;
  int64_t begin;
  int count;
};

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
  return ti;
}

template <int PREC>
__device__ __forceinline__ bool same_weights(const DevModel *a, const DevModel *b) {
  return a == b || (a && b && a->tc_img[PREC] == b->tc_img[PREC]);
}

__device__ __forceinline__ uint32_t img_w0() { return 0; }
__device__ __forceinline__ uint32_t img_wh(int l) { return kTcW0HalfBytes + (l - 1) * kTcWhHalfBytes; }

// H chunk epilogue for one warp: 32 rows x 32 columns of fp32 accumulator (+bias, ReLU)
// -> packed fp16/bf16 -> H (K-major core-matrix layout).
template <int PREC>
__device__ __forceinline__ void epi_to_h(const uint32_t (&r)[32], const float *bl, uint32_t col0,
                                         uint32_t hrow_addr) {
#pragma unroll
  for (int gq = 0; gq < 4; ++gq) {
    uint32_t p[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int c = gq * 8 + e * 2;
      const float v0 = __uint_as_float(r[c]) + bl[col0 + c];
      const float v1 = __uint_as_float(r[c + 1]) + bl[col0 + c + 1];
      p[e] = PREC == 0 ? ptx::relu_pack_f16(v0, v1) : ptx::relu_pack_bf16(v0, v1);
    }
    ptx::st_shared_v4(hrow_addr + ((col0 >> 3) + gq) * kLboR128, p[0], p[1], p[2], p[3]);
  }
}

// Last hidden layer: ReLU(acc + b) in fp32, accumulated straight into the two logits.
__device__ __forceinline__ void epi_to_logits(const uint32_t (&r)[32], const float *bl,
                                              const float *wo, uint32_t col0, float &p0,
                                              float &p1) {
#pragma unroll
  for (int c = 0; c < 32; ++c) {
    float h = __uint_as_float(r[c]) + bl[col0 + c];
    h = h > 0.0f ? h : 0.0f;
    p0 = fmaf(h, wo[col0 + c], p0);
    p1 = fmaf(h, wo[kHidden + col0 + c], p1);
  }
}

template <int PREC, int IN_KIND>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
mlp_tc_kernel(const void *__restrict__ in, const __grid_constant__ TileSched ts, int nh_layout,
              uint8_t *__restrict__ decisions, float *__restrict__ logits) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const Layout L = tc_layout(nh_layout);
  const uint32_t sbase = ptx::smem_u32(smem);
  const uint32_t bar0 = sbase + L.bar;
  auto bar = [&](uint32_t slot) { return bar0 + slot * 8; };
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ptx::cluster_ctarank();
  const uint32_t cid = ptx::cluster_id_x(), ncl = ptx::num_clusters_x();

  const int64_t n_tiles = ts.n_tiles_dev ? (int64_t)*ts.n_tiles_dev : ts.n_tiles;
  const int64_t t_begin = n_tiles * cid / ncl;
  const int64_t t_end = n_tiles * (cid + 1) / ncl;

  if (threadIdx.x == 0) {
    ptx::mbar_init(bar(B_WLOAD), 1);
    ptx::mbar_init(bar(B_WREADY), 2);            // one arrive per CTA loader
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(bar(B_XFULL + i), 2);       // one arrive per CTA digitiser group
      ptx::mbar_init(bar(B_XEMPTY + i), 1);      // tcgen05.commit (multicast)
      ptx::mbar_init(bar(B_DFULL + i), 1);       // tcgen05.commit (multicast)
      ptx::mbar_init(bar(B_TEMPTY + i), 16);     // 8 epilogue warps x 2 CTAs
    }
    for (int i = 0; i < 4; ++i) ptx::mbar_init(bar(B_HREADY + i), 16);
    ptx::mbar_init(bar(B_WFREE), 1);             // tcgen05.commit (multicast)
    ptx::fence_mbar_init();
  }
  if (warp == 0) {
    ptx::tmem_alloc_cg2(sbase + L.bar + kTmemSlot, 512);
    ptx::tmem_relinquish_cg2();
  }
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + L.bar + kTmemSlot);

  if (warp == 0) {
    // ================= weight loader (both CTAs) =================
    if (lane == 0) {
      const DevModel *cur = nullptr;
      uint32_t wl_phase = 0, wf_phase = 0;
      const uint32_t wready_leader = ptx::mapa(bar(B_WREADY), 0);
      for (int64_t t = t_begin; t < t_end; ++t) {
        const TileInfo ti = tile_info(ts, t);
        if (same_weights<PREC>(ti.model, cur)) continue;
        // Model switch: every MMA reading the old weights must have completed. The MMA
        // thread commits B_WFREE once per switch, after the old model's last MMA; it cannot
        // commit the next one before this loader has signalled B_WREADY (lag <= 1 phase).
        if (cur) {
          ptx::mbar_wait(bar(B_WFREE), wf_phase);
          wf_phase ^= 1;
        }
        const uint32_t bytes = ti.model->tc_img_bytes;
        const uint8_t *src = ti.model->tc_img[PREC] + (size_t)rank * bytes;
        ptx::mbar_arrive_expect_tx(bar(B_WLOAD), bytes);
        for (uint32_t off = 0; off < bytes; off += 32768) {
          const uint32_t len = (bytes - off) < 32768 ? (bytes - off) : 32768;
          ptx::bulk_g2s(sbase + off, src + off, len, bar(B_WLOAD));
        }
        ptx::mbar_wait(bar(B_WLOAD), wl_phase);
        wl_phase ^= 1;
        ptx::mbar_arrive_cluster(wready_leader);
        cur = ti.model;
      }
    }
  } else if (warp == 1) {
    // ================= MMA issuer (leader CTA, one thread) =================
    if (rank == 0 && lane == 0) {
      const uint32_t idesc = ptx::umma_idesc_f16(PREC, 256, 256);
      const DevModel *cur = nullptr;
      uint32_t w_phase = 0, g = 0, h_phase = 0, t_phase = 0;  // h/t_phase: one bit per slot
      uint32_t uses[2] = {0, 0};
      int64_t it = 0;
      auto acquire_buf = [&](uint32_t b) {  // accumulator b must be drained by the epilogues
        if (uses[b]++ > 0) {
          ptx::mbar_wait(bar(B_TEMPTY + b), (t_phase >> b) & 1);
          t_phase ^= (1u << b);
        }
      };
      for (int64_t t = t_begin; t < t_end; ++t, ++it) {
        const TileInfo ti = tile_info(ts, t);
        if (!same_weights<PREC>(ti.model, cur)) {
          ptx::mbar_wait(bar(B_WREADY), w_phase);
          w_phase ^= 1;
          cur = ti.model;
        }
        const int nh = ti.model->nh;
        const uint32_t xb = (uint32_t)(it & 1);
        {  // layer 0: D = X[128(x2) x 32] * W0^T
          const uint32_t b = g & 1;
          acquire_buf(b);
          ptx::mbar_wait(bar(B_XFULL + xb), (uint32_t)((it >> 1) & 1));
          ptx::tc_fence_after();
          const uint32_t d = tmem + b * 256;
          const uint32_t xa = sbase + L.x + xb * kXBytes;
#pragma unroll
          for (uint32_t s = 0; s < kTcK0 / 16; ++s)
            ptx::mma_f16_cg2(d, ptx::umma_desc(xa + s * 2 * kLboR128, kLboR128, 128),
                             ptx::umma_desc(sbase + img_w0() + s * 2 * kLboR128, kLboR128, 128),
                             idesc, s);
          ptx::mma_commit_cg2(bar(B_XEMPTY + xb), 0x3);
          ptx::mma_commit_cg2(bar(B_DFULL + b), 0x3);
          ++g;
        }
        for (int l = 1; l < nh; ++l) {  // hidden layers 1..nh-1 (K = 256)
          const uint32_t b = g & 1;
          acquire_buf(b);
          ptx::tc_fence_after();
          const uint32_t d = tmem + b * 256;
          for (uint32_t kc = 0; kc < 4; ++kc) {
            ptx::mbar_wait(bar(B_HREADY + kc), (h_phase >> kc) & 1);
            h_phase ^= (1u << kc);
            ptx::tc_fence_after();
#pragma unroll
            for (uint32_t s = 0; s < 4; ++s) {
              const uint32_t ks = kc * 4 + s;
              ptx::mma_f16_cg2(d, ptx::umma_desc(sbase + L.h + ks * 2 * kLboR128, kLboR128, 128),
                               ptx::umma_desc(sbase + img_wh(l) + ks * 2 * kLboR128, kLboR128, 128),
                               idesc, ks);
            }
          }
          ptx::mma_commit_cg2(bar(B_DFULL + b), 0x3);
          ++g;
        }
        if (t + 1 < t_end && !same_weights<PREC>(tile_info(ts, t + 1).model, cur))
          ptx::mma_commit_cg2(bar(B_WFREE), 0x3);  // old weights no longer read
      }
    }
  } else if (warp < 4) {
    // ================= digitisers: raw -> X (fp16/bf16 digits), 2 rows per thread ========
    const uint32_t d = threadIdx.x - 64;  // 0..63
    const uint32_t xfull_leader0 = ptx::mapa(bar(B_XFULL), 0);
    int64_t it = 0;
    for (int64_t t = t_begin; t < t_end; ++t, ++it) {
      const TileInfo ti = tile_info(ts, t);
      const uint32_t xb = (uint32_t)(it & 1);
      ptx::mbar_wait(bar(B_XEMPTY + xb), (uint32_t)(((it >> 1) & 1) ^ 1));
      const uint32_t xs = sbase + L.x + xb * kXBytes;
#pragma unroll
      for (int half = 0; half < 2; ++half) {
        const uint32_t r = d + 64 * half;
        const int pos = (int)(rank * 128 + r);
        uint32_t w[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) w[i] = 0;
        if (pos < ti.count) {
          const int64_t p = ti.begin + pos;
          const int64_t io = ts.perm ? (int64_t)ts.perm[p] : p;
          if (IN_KIND == LAKE_IN_RAW) {
            const uint32_t *src = reinterpret_cast<const uint32_t *>(in) + io * 9;
            uint32_t rec[9];
#pragma unroll
            for (int f = 0; f < 9; ++f) rec[f] = __ldg(src + f);
            // digit values 0..9 are exact in fp16 and bf16
            digitize_record(rec, [&](int k, uint32_t dg) {
              const float v = (float)dg;
              const uint16_t hbits = PREC == 0 ? __half_as_ushort(__float2half_rn(v))
                                               : __bfloat16_as_ushort(__float2bfloat16_rn(v));
              w[k >> 1] |= (uint32_t)hbits << ((k & 1) * 16);
            });
          } else {
            const uint4 *src = reinterpret_cast<const uint4 *>(
                reinterpret_cast<const uint8_t *>(in) + io * 32);
            const uint4 v0 = __ldg(src), v1 = __ldg(src + 1);
            const uint32_t b[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
#pragma unroll
            for (int k = 0; k < 31; ++k) {
              const float v = (float)((b[k >> 2] >> ((k & 3) * 8)) & 0xFFu);
              const uint16_t hbits = PREC == 0 ? __half_as_ushort(__float2half_rn(v))
                                               : __bfloat16_as_ushort(__float2bfloat16_rn(v));
              w[k >> 1] |= (uint32_t)hbits << ((k & 1) * 16);
            }
          }
        }
#pragma unroll
        for (int kg = 0; kg < 4; ++kg)
          ptx::st_shared_v4(xs + kg * kLboR128 + r * 16, w[kg * 4 + 0], w[kg * 4 + 1],
                            w[kg * 4 + 2], w[kg * 4 + 3]);
      }
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(1, 64);
      if (d == 0) ptx::mbar_arrive_cluster(xfull_leader0 + xb * 8);
    }
  } else {
    // ================= epilogue =================
    const uint32_t et = threadIdx.x - 128;  // 0..255
    const uint32_t q = warp & 3;            // TMEM lane quadrant this warp may access
    const uint32_t hh = (warp - 4) >> 2;    // which 32-column half of each 64-column chunk
    const uint32_t row = q * 32 + lane;     // row within this CTA's 128
    const uint32_t hready_leader0 = ptx::mapa(bar(B_HREADY), 0);
    const uint32_t tempty_leader0 = ptx::mapa(bar(B_TEMPTY), 0);
    const uint32_t hrow = sbase + L.h + row * 16;
    float *prm = reinterpret_cast<float *>(smem + L.prm);
    float *red = reinterpret_cast<float *>(smem + L.red);
    const DevModel *cur = nullptr;
    uint32_t g = 0, d_phase = 0;  // d_phase: bit b
    int64_t it = 0;
    for (int64_t t = t_begin; t < t_end; ++t, ++it) {
      const TileInfo ti = tile_info(ts, t);
      const int nh = ti.model->nh;
      if (ti.model != cur) {
        // stage this model's fp32 biases | W_out | b_out (contiguous in its FP32 image)
        const uint32_t nf4 = (nh * kHidden + 2 * kHidden + 4) / 4;
        ptx::named_bar_sync(2, 256);
        const float4 *src = reinterpret_cast<const float4 *>(ti.model->b[0]);
        for (uint32_t i = et; i < nf4; i += 256) reinterpret_cast<float4 *>(prm)[i] = __ldg(src + i);
        ptx::named_bar_sync(2, 256);
        cur = ti.model;
      }
      const float *wo = prm + nh * kHidden;
      for (int l = 0; l < nh; ++l) {
        const uint32_t b = g & 1;
        ptx::mbar_wait(bar(B_DFULL + b), (d_phase >> b) & 1);
        d_phase ^= (1u << b);
        ptx::tc_fence_after();
        const uint32_t tbase = tmem + ((q * 32) << 16) + b * 256 + hh * 32;
        const float *bl = prm + l * kHidden;
        uint32_t ra[32], rb[32];
        ptx::tmem_ld_32x32b_x32(tbase, ra);
        ptx::tmem_ld_wait();
        if (l + 1 < nh) {
          // hidden layer feeding another MMA: 4 chunks of 64 columns, TMEM loads of the next
          // chunk in flight while the current one is converted and stored
#pragma unroll
          for (uint32_t kc = 0; kc < 4; ++kc) {
            const uint32_t col0 = kc * 64 + hh * 32;
            if (kc + 1 < 4) {
              if (kc & 1) ptx::tmem_ld_32x32b_x32(tbase + (kc + 1) * 64, ra);
              else ptx::tmem_ld_32x32b_x32(tbase + (kc + 1) * 64, rb);
            }
            if (kc & 1) epi_to_h<PREC>(rb, bl, col0, hrow);
            else epi_to_h<PREC>(ra, bl, col0, hrow);
            ptx::fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive_cluster(hready_leader0 + kc * 8);
            if (kc + 1 < 4) ptx::tmem_ld_wait();
          }
        } else {
          // last hidden layer: fold the 2-neuron output layer (fp32, CUDA cores)
          float p0 = 0.0f, p1 = 0.0f;
#pragma unroll
          for (uint32_t kc = 0; kc < 4; ++kc) {
            const uint32_t col0 = kc * 64 + hh * 32;
            if (kc + 1 < 4) {
              if (kc & 1) ptx::tmem_ld_32x32b_x32(tbase + (kc + 1) * 64, ra);
              else ptx::tmem_ld_32x32b_x32(tbase + (kc + 1) * 64, rb);
            }
            if (kc & 1) epi_to_logits(rb, bl, wo, col0, p0, p1);
            else epi_to_logits(ra, bl, wo, col0, p0, p1);
            if (kc + 1 < 4) ptx::tmem_ld_wait();
          }
          float *rd = red + (it & 1) * 256 + row * 2;
          if (hh == 1) {
            rd[0] = p0;
            rd[1] = p1;
          }
          ptx::named_bar_sync(3 + q, 64);  // the two warps sharing this quadrant
          if (hh == 0) {
            const float l0 = p0 + rd[0] + wo[2 * kHidden + 0];
            const float l1 = p1 + rd[1] + wo[2 * kHidden + 1];
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
        }
        // accumulator b fully read by this warp
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive_cluster(tempty_leader0 + b * 8);
        ++g;
      }
    }
  }

  __syncwarp();  // reconverge role lanes before the .aligned cluster barrier
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_cg2(tmem, 512);
  }
}

template <int PREC, int IN_KIND>
cudaError_t launch_t(const void *in, const TileSched &ts, int nh_layout, uint8_t *dec,
                     float *logits, cudaStream_t s, int grid) {
  const Layout L = tc_layout(nh_layout);
  static bool attr_set[64] = {};
  int dev = 0;
  cudaGetDevice(&dev);
  if (!attr_set[dev & 63]) {
    cudaError_t e = cudaFuncSetAttribute(mlp_tc_kernel<PREC, IN_KIND>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)tc_layout(kMaxHiddenLayers).total);
    if (e != cudaSuccess) return e;
    attr_set[dev & 63] = true;
  }
  mlp_tc_kernel<PREC, IN_KIND><<<grid, kThreads, L.total, s>>>(in, ts, nh_layout, dec, logits);
  return cudaGetLastError();
}

}  // namespace

size_t tc_smem_bytes(int nh_layout) { return tc_layout(nh_layout).total; }

cudaError_t launch_mlp_tc(const void *in, int in_kind, int prec, const TileSched &ts, int nh,
                          uint8_t *decisions, float *logits, cudaStream_t s, int device) {
  static int sms_cache[64] = {};
  int sms = sms_cache[device & 63];
  if (!sms) {
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    sms_cache[device & 63] = sms;
  }
  const int64_t max_clusters = sms / 2;
  const int64_t clusters = ts.n_tiles < max_clusters ? ts.n_tiles : max_clusters;
  if (clusters <= 0) return cudaSuccess;
  const int grid = (int)(clusters * 2);
  cudaError_t e;
  if (prec == 0)
    e = in_kind == LAKE_IN_RAW ? launch_t<0, LAKE_IN_RAW>(in, ts, nh, decisions, logits, s, grid)
                               : launch_t<0, LAKE_IN_DIGITS>(in, ts, nh, decisions, logits, s, grid);
  else
    e = in_kind == LAKE_IN_RAW ? launch_t<1, LAKE_IN_RAW>(in, ts, nh, decisions, logits, s, grid)
                               : launch_t<1, LAKE_IN_DIGITS>(in, ts, nh, decisions, logits, s, grid);
  count_launch();
  return e;
}

}  // namespace lake
