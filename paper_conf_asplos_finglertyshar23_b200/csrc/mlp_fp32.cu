// mlp_fp32.cu — fused digitise -> MLP -> argmax on CUDA cores in FP32, bit-exact with the
// oracle under reading R15: every output accumulates from +0.0f with one
// __fmaf_rn per input in ascending k, then one __fadd_rn of the bias, then ReLU as
// (z > 0 ? z : +0). No split-K, no tree reduction, no FTZ, no contraction (--fmad=false).
//
// Network: "two layers with 256 and 2 neurons" (+1 / +2 hidden layers), §7.1
// P:1168-1177. Batch scoring (score_features, Table 1).
//
// Mapping: a CTA (256 threads) owns an M-I/O tile (M = 64, or 16 for small single-model
// batches, where latency rather than throughput matters). Hidden layers are register-tiled
// GEMMs: thread (tr = warp, tc = lane) owns RM = M/8 rows {h*M/2 + tr*RM/2 + i} x 8 columns
// {tc + 32*jj}.
// Each accumulator is summed over k strictly in order (that is what a K-loop GEMM does),
// so the tiling changes nothing numerically. Activations live transposed in SMEM
// (act[k][row], row stride 68 floats: broadcast A reads, conflict-free epilogue stores);
// weights stream through a 2-stage cp.async pipeline in 16-row chunks of W^T, activations
// are updated in place (two CTAs fit per SM: 16 warps), and W^T columns
// were permuted at load time so each thread's 8 columns are two float4s.
// The 2-wide output layer is one sequential fmaf chain per (row, class).
#include <cuda_pipeline.h>

#include "digitize.cuh"
#include <atomic>

#include "lake_internal.h"
#include "lake_ptx.cuh"

namespace lake {
namespace {

#ifndef LAKE_F32_UNROLL
#define LAKE_F32_UNROLL 2  // no register spill at 2 CTAs/SM (4: 32-B spill, same speed)
#endif
constexpr int kF32Unroll = LAKE_F32_UNROLL;  // k-loop unroll of the RM = 8 tile
#ifndef LAKE_F32_ACT_BUFS
#define LAKE_F32_ACT_BUFS 1
#endif
constexpr int kF32ActBufs = LAKE_F32_ACT_BUFS;
#ifndef LAKE_F32_CTAS
#define LAKE_F32_CTAS 2  // CTAs per SM (<= 128 registers; A/B: 1 -> 2 CTAs +3% NN+2, +36% NN)
#endif  // 1: in place (frees SMEM for KC = 64)

#ifndef LAKE_F32_FFMA2
#define LAKE_F32_FFMA2 0  // 1: hot loop on fma.rn.f32x2 (A/B)
#endif
#ifndef LAKE_F32_PF
#define LAKE_F32_PF 0  // 1: register double buffer of the next k-step (A/B: 6.74 vs 5.76 ms)
#endif
#ifndef LAKE_F32_WIDE_KC
#define LAKE_F32_WIDE_KC 32
#endif
// Register tile RM rows x RN columns per thread, 256 threads: CG column groups (lanes across
// the 256 columns) x RG row groups, M = RG * RM rows per tile.
//   RM 2, RN 8  (M 16):  small single-model batches (latency)
//   RM 8, RN 8  (M 64):  two CTAs per SM (round 1)
//   RM 8, RN 16 (M 128): one CTA per SM, 128 accumulators per thread: per k-step 6 shared
//                        loads feed 128 FFMAs (RN 8: 4 feed 64), half the SMEM wavefronts
//                        per FMA and fewer barriers per FMA (32-row weight chunks)
template <int RM, int RN>
struct F32Cfg {
  static constexpr int T = RM == 4 ? 512 : kF32Threads;  // threads (RM 4: 16 warps per CTA)
  static constexpr int CG = 256 / RN;                    // column groups
  static constexpr int RG = T / CG;                      // row groups
  static constexpr int M = RG * RM;                      // rows per tile
  static constexpr int HR = RM / 2;                      // rows per thread per half-tile
  static constexpr int NF4 = RN / 4;                     // float4 weight loads per k-step
  // activation row stride: float4-aligned with a 4-float pad for RM = 8 (conflict-free
  // float4 epilogue stores), odd for RM = 2 (conflict-free scalar stores)
  static constexpr int S = RM >= 4 ? M + 4 : M + 1;
  // rows of W^T per pipeline stage: RN 8 / RM 8 uses 16 (LAKE_F32_KC) so that two CTAs fit
  // per SM (A/B on B200: 1 CTA/SM with 64-row chunks 6.37 ms, 2 CTAs/SM with 16-row chunks
  // 6.19 ms, C3 NN+2)
  static constexpr int KC = RN == 16 ? LAKE_F32_WIDE_KC : (RM == 8 ? kF32KChunk : 16);
  static constexpr int CTAS = RN == 16 ? 1 : LAKE_F32_CTAS;  // resident CTAs per SM
};
#ifndef LAKE_F32_RM
#define LAKE_F32_RM 8  // rows per thread of the full-size tile: 8 (256 threads) or 4 (512 threads)
#endif
constexpr int kF32TileRM = LAKE_F32_RM;
static_assert(F32Cfg<kF32TileRM, kF32TileRN>::M == kF32TileM, "multi-model FP32 tile rows");

template <int RM, int RN>
struct F32Smem {
  // transposed activations, updated in place: a layer's outputs are written only after
  // the __syncthreads that closes its last K chunk, i.e. once every input has been read
  float act[kF32ActBufs][kHidden][F32Cfg<RM, RN>::S];
  float w[2][F32Cfg<RM, RN>::KC][kHidden];   // W^T chunk staging (permuted columns)
  float wout[2][kHidden];
  float bout[4];
  int32_t rows[F32Cfg<RM, RN>::M];           // I/O index per tile row, -1 = padding
};

template <int T>
__device__ __forceinline__ void stage_chunk(float (*dst)[kHidden], const float *src, int rows) {
  // rows x 256 floats, contiguous in global; 16-byte cp.async per thread-iteration.
  const int n16 = rows * kHidden / 4;
  for (int i = threadIdx.x; i < n16; i += T) {
    __pipeline_memcpy_async(reinterpret_cast<float4 *>(&dst[0][0]) + i,
                            reinterpret_cast<const float4 *>(src) + i, 16);
  }
  __pipeline_commit();
}

template <int IN_KIND, int RM, int RN>
__global__ void __launch_bounds__(F32Cfg<RM, RN>::T, F32Cfg<RM, RN>::CTAS)
mlp_fp32_kernel(const void *__restrict__ in, const __grid_constant__ TileSched ts,
                uint8_t *__restrict__ decisions,
                float *__restrict__ logits) {
  using C = F32Cfg<RM, RN>;
  constexpr int M = C::M, S = C::S, HR = C::HR, KC = C::KC, CG = C::CG, NF4 = C::NF4, T = C::T;
  extern __shared__ __align__(16) uint8_t smem_raw[];
  F32Smem<RM, RN> &sm = *reinterpret_cast<F32Smem<RM, RN> *>(smem_raw);
  const int tid = threadIdx.x;
  const int tr = tid / CG;   // row group
  const int tc = tid % CG;   // column group
  const int64_t n_tiles = ts.n_tiles_dev ? (int64_t)*ts.n_tiles_dev : ts.n_tiles;

  for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
    const DevModel *mp = ts.tile_model ? &ts.table[ts.tile_model[tile]] : &ts.model;
    const int nh = mp->nh;
    int64_t begin;
    int count;
    if (ts.tile_model) {
      begin = ts.tile_begin[tile];
      count = ts.tile_count[tile];
    } else {
      begin = tile * M;
      count = (int)((ts.n - begin) < M ? (ts.n - begin) : M);
    }
    __syncthreads();  // previous tile's output layer is done with act[] / wout
    // ---- rows, digits -> act[0][k][r] (k < 32, row 31 = 0) --------------------------
    if (tid < M) {
      int32_t io = -1;
      if (tid < count) io = ts.perm ? ts.perm[begin + tid] : (int32_t)(begin + tid);
      sm.rows[tid] = io;
      float (*a0)[S] = sm.act[0];
      if (io < 0) {
        for (int k = 0; k < 32; ++k) a0[k][tid] = 0.0f;
      } else if (IN_KIND == LAKE_IN_RAW) {
        const uint32_t *r = reinterpret_cast<const uint32_t *>(in) + (int64_t)io * 9;
        uint32_t rec[9];
#pragma unroll
        for (int f = 0; f < 9; ++f) rec[f] = __ldg(r + f);
        digitize_record(rec, [&](int pos, uint32_t d) { a0[pos][tid] = (float)d; });
        a0[31][tid] = 0.0f;
      } else {
        const uint4 *p = reinterpret_cast<const uint4 *>(
            reinterpret_cast<const uint8_t *>(in) + (int64_t)io * 32);
        uint4 v0 = __ldg(p), v1 = __ldg(p + 1);
        uint32_t w[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
#pragma unroll
        for (int k = 0; k < 32; ++k) a0[k][tid] = (float)((w[k >> 2] >> ((k & 3) * 8)) & 0xFFu);
      }
    } else {
      // output-layer weights for this tile's model (the threads not digitising)
      for (int i = tid - M; i <= 2 * kHidden / 4; i += T - M) {
        if (i < 2 * kHidden / 4)
          reinterpret_cast<float4 *>(&sm.wout[0][0])[i] =
              __ldg(reinterpret_cast<const float4 *>(mp->wout) + i);
        else {
          sm.bout[0] = __ldg(mp->bout);
          sm.bout[1] = __ldg(mp->bout + 1);
        }
      }
    }
    // ---- hidden layers -----------------------------------------------------------------
    for (int l = 0; l < nh; ++l) {
      const int K = (l == 0) ? kInputs : kHidden;         // strict: layer 0 sums 31 terms
      const int Kst = (l == 0) ? 32 : kHidden;            // staged rows (row 31 is zero)
      const float *wt = mp->wt[l];
      const float (*ain)[S] = sm.act[kF32ActBufs == 2 ? (l & 1) : 0];
      float (*aout)[S] = sm.act[kF32ActBufs == 2 ? ((l + 1) & 1) : 0];
      float acc[RM][RN];
#pragma unroll
      for (int i = 0; i < RM; ++i)
#pragma unroll
        for (int j = 0; j < RN; ++j) acc[i][j] = 0.0f;
#if LAKE_F32_FFMA2
      // paired accumulators (columns 2jp, 2jp+1 of row i): one fma.rn.f32x2 does two FMAs,
      // each rounded exactly as __fmaf_rn (bit-exact); halves the FFMA instruction count of
      // the issue-bound hot loop
      uint64_t acc2[RM][RN / 2];
#pragma unroll
      for (int i = 0; i < RM; ++i)
#pragma unroll
        for (int jp = 0; jp < RN / 2; ++jp) acc2[i][jp] = 0ull;
#endif
      const int nch = (Kst + KC - 1) / KC;  // layer 0 stages its 32 rows even when KC > 32
      stage_chunk<T>(sm.w[0], wt, Kst < KC ? Kst : KC);
      for (int c = 0; c < nch; ++c) {
        if (c + 1 < nch) {
          const int rows = (Kst - (c + 1) * KC) < KC ? (Kst - (c + 1) * KC) : KC;
          stage_chunk<T>(sm.w[(c + 1) & 1], wt + (int64_t)(c + 1) * KC * kHidden, rows);
          __pipeline_wait_prior(1);
        } else {
          __pipeline_wait_prior(0);
        }
        __syncthreads();
        const float (*wc)[kHidden] = sm.w[c & 1];
        const int kmax = (K - c * KC) < KC ? (K - c * KC) : KC;
        // one k-step's operands: RM activations (broadcast float4 reads) and RN weights
        auto load_ops = [&](int kk, float (&av)[RM], float (&bv)[RN]) {
          const int k = c * KC + kk;
          if constexpr (HR == 4) {
            const float4 a0 = *reinterpret_cast<const float4 *>(&ain[k][tr * 4]);
            const float4 a1 = *reinterpret_cast<const float4 *>(&ain[k][M / 2 + tr * 4]);
            av[0] = a0.x; av[1] = a0.y; av[2] = a0.z; av[3] = a0.w;
            av[4] = a1.x; av[5] = a1.y; av[6] = a1.z; av[7] = a1.w;
          } else if constexpr (HR == 2 && RM == 4) {
            const float2 a0 = *reinterpret_cast<const float2 *>(&ain[k][tr * 2]);
            const float2 a1 = *reinterpret_cast<const float2 *>(&ain[k][M / 2 + tr * 2]);
            av[0] = a0.x; av[1] = a0.y; av[2] = a1.x; av[3] = a1.y;
          } else {
#pragma unroll
            for (int i = 0; i < HR; ++i) {
              av[i] = ain[k][tr * HR + i];
              av[HR + i] = ain[k][M / 2 + tr * HR + i];
            }
          }
#pragma unroll
          for (int f = 0; f < NF4; ++f) {
            const float4 b4 = *reinterpret_cast<const float4 *>(&wc[kk][f * 4 * CG + tc * 4]);
            bv[4 * f] = b4.x; bv[4 * f + 1] = b4.y; bv[4 * f + 2] = b4.z; bv[4 * f + 3] = b4.w;
          }
        };
#if LAKE_F32_PF == 2
        // software-pipelined with two explicit operand sets (no register copies) and no
        // branches around the loads (a predicated load was sunk below the FFMAs it was meant
        // to overlap): k-step kk+1's shared loads are issued before kk's FFMAs; the last
        // iteration's look-ahead load re-reads a valid row and is not used
        {
          float a0[RM], b0[RN], a1[RM], b1[RN];
          load_ops(0, a0, b0);
          int kk = 0;
          for (; kk + 1 < kmax; kk += 2) {
            load_ops(kk + 1, a1, b1);
#pragma unroll
            for (int i = 0; i < RM; ++i)
#pragma unroll
              for (int j = 0; j < RN; ++j) acc[i][j] = __fmaf_rn(a0[i], b0[j], acc[i][j]);
            load_ops(kk + 2 < kmax ? kk + 2 : kmax - 1, a0, b0);
#pragma unroll
            for (int i = 0; i < RM; ++i)
#pragma unroll
              for (int j = 0; j < RN; ++j) acc[i][j] = __fmaf_rn(a1[i], b1[j], acc[i][j]);
          }
          if (kk < kmax) {  // odd kmax (layer 0: 31 terms): a0/b0 hold k-step kk
#pragma unroll
            for (int i = 0; i < RM; ++i)
#pragma unroll
              for (int j = 0; j < RN; ++j) acc[i][j] = __fmaf_rn(a0[i], b0[j], acc[i][j]);
          }
        }
#elif LAKE_F32_PF
        // software-pipelined: k-step kk+1's shared loads are in flight during kk's FFMAs (with
        // two warps per scheduler at RN 16, their latency was the top stall)
        float av[RM], bv[RN];
        load_ops(0, av, bv);
#pragma unroll kF32Unroll
        for (int kk = 0; kk < kmax; ++kk) {
          float an[RM], bn[RN];
          if (kk + 1 < kmax) load_ops(kk + 1, an, bn);
#pragma unroll
          for (int i = 0; i < RM; ++i)
#pragma unroll
            for (int j = 0; j < RN; ++j) acc[i][j] = __fmaf_rn(av[i], bv[j], acc[i][j]);
#pragma unroll
          for (int i = 0; i < RM; ++i) av[i] = an[i];
#pragma unroll
          for (int j = 0; j < RN; ++j) bv[j] = bn[j];
        }
#else
#pragma unroll kF32Unroll
        for (int kk = 0; kk < kmax; ++kk) {
          float av[RM], bv[RN];
          load_ops(kk, av, bv);
#if LAKE_F32_FFMA2
          uint64_t bp[RN / 2];
#pragma unroll
          for (int jp = 0; jp < RN / 2; ++jp) bp[jp] = ptx::pack_f32x2(bv[2 * jp], bv[2 * jp + 1]);
#pragma unroll
          for (int i = 0; i < RM; ++i) {
            const uint64_t ap = ptx::pack_f32x2(av[i], av[i]);
#pragma unroll
            for (int jp = 0; jp < RN / 2; ++jp) ptx::fma_f32x2(acc2[i][jp], ap, bp[jp]);
          }
#else
#pragma unroll
          for (int i = 0; i < RM; ++i)
#pragma unroll
            for (int j = 0; j < RN; ++j) acc[i][j] = __fmaf_rn(av[i], bv[j], acc[i][j]);
#endif
        }
#endif
        __syncthreads();
      }
#if LAKE_F32_FFMA2
#pragma unroll
      for (int i = 0; i < RM; ++i)
#pragma unroll
        for (int jp = 0; jp < RN / 2; ++jp) ptx::unpack_f32x2(acc2[i][jp], acc[i][2 * jp], acc[i][2 * jp + 1]);
#endif
      // epilogue: z = acc + b (one rounding), ReLU, store transposed
      const float *bias = mp->b[l];
#pragma unroll
      for (int jj = 0; jj < RN; ++jj) {
        // staged position p of this accumulator column -> its neuron (the load-time column
        // permutation: position 128 b + 4 t + q holds neuron t + 32 (q + 4 b), t < 32)
        const int p = (jj / 4) * 4 * CG + tc * 4 + (jj % 4);
        const int j = ((p >> 2) & 31) + 32 * ((p & 3) + 4 * (p >> 7));
        const float bj = __ldg(bias + j);
        float h[RM];
#pragma unroll
        for (int i = 0; i < RM; ++i) {
          const float z = __fadd_rn(acc[i][jj], bj);
          h[i] = (z > 0.0f) ? z : 0.0f;
        }
        if constexpr (HR == 4) {
          *reinterpret_cast<float4 *>(&aout[j][tr * 4]) = make_float4(h[0], h[1], h[2], h[3]);
          *reinterpret_cast<float4 *>(&aout[j][M / 2 + tr * 4]) =
              make_float4(h[4], h[5], h[6], h[7]);
        } else if constexpr (HR == 2 && RM == 4) {
          *reinterpret_cast<float2 *>(&aout[j][tr * 2]) = make_float2(h[0], h[1]);
          *reinterpret_cast<float2 *>(&aout[j][M / 2 + tr * 2]) = make_float2(h[2], h[3]);
        } else {
#pragma unroll
          for (int i = 0; i < HR; ++i) {
            aout[j][tr * HR + i] = h[i];
            aout[j][M / 2 + tr * HR + i] = h[HR + i];
          }
        }
      }
      __syncthreads();
    }
    // ---- output layer (2 neurons, identity) + decision ------------------------------------
    if (tid < 2 * M) {
      const int r = tid >> 1, c = tid & 1;
      const float (*h)[S] = sm.act[kF32ActBufs == 2 ? (nh & 1) : 0];
      float acc = 0.0f;
#pragma unroll 8
      for (int k = 0; k < kHidden; ++k) acc = __fmaf_rn(h[k][r], sm.wout[c][k], acc);
      const float z = __fadd_rn(acc, sm.bout[c]);
      const float other = __shfl_xor_sync(0xffffffffu, z, 1);
      const int32_t io = sm.rows[r];
      if (io >= 0) {
        if (logits) logits[(int64_t)io * 2 + c] = z;
        if (c == 0) decisions[io] = (other > z) ? 1 : 0;  // logit1 > logit0; ties/NaN -> 0
      }
    }
  }
}

template <int IN_KIND, int RM, int RN>
cudaError_t launch_rm(const void *in, const TileSched &ts, uint8_t *decisions, float *logits,
                      cudaStream_t s, int64_t grid) {
  const size_t smem = sizeof(F32Smem<RM, RN>);
  static std::atomic<bool> attr_set[64];  // shared by host threads
  int dev = 0;
  cudaGetDevice(&dev);
  if (!attr_set[dev & 63].load(std::memory_order_acquire)) {
    cudaError_t e = cudaFuncSetAttribute(mlp_fp32_kernel<IN_KIND, RM, RN>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set[dev & 63].store(true, std::memory_order_release);
  }
  mlp_fp32_kernel<IN_KIND, RM, RN><<<(unsigned)grid, F32Cfg<RM, RN>::T, smem, s>>>(in, ts, decisions,
                                                                                 logits);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_mlp_fp32(const void *in, int in_kind, const TileSched &ts_in,
                            uint8_t *decisions, float *logits, cudaStream_t s, int device) {
  static std::atomic<int> sms_cache[64];
  int sms = sms_cache[device & 63].load(std::memory_order_relaxed);
  if (!sms) {
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    sms_cache[device & 63].store(sms, std::memory_order_relaxed);
  }
  TileSched ts = ts_in;
  // small single-model batches: 16-row tiles (4x less work per tile on the critical path)
  const bool small = ts.tile_model == nullptr && ts.n <= (int64_t)16 * sms;
  if (small) ts.n_tiles = (ts.n + 15) / 16;
  const int64_t cap = (int64_t)sms * (small ? F32Cfg<2, 8>::CTAS : F32Cfg<kF32TileRM, kF32TileRN>::CTAS);
  const int64_t grid = ts.n_tiles < cap ? ts.n_tiles : cap;
  if (grid <= 0) return cudaSuccess;
  cudaError_t e;
  if (in_kind == LAKE_IN_RAW)
    e = small ? launch_rm<LAKE_IN_RAW, 2, 8>(in, ts, decisions, logits, s, grid)
              : launch_rm<LAKE_IN_RAW, kF32TileRM, kF32TileRN>(in, ts, decisions, logits, s, grid);
  else
    e = small ? launch_rm<LAKE_IN_DIGITS, 2, 8>(in, ts, decisions, logits, s, grid)
              : launch_rm<LAKE_IN_DIGITS, kF32TileRM, kF32TileRN>(in, ts, decisions, logits, s, grid);
  count_launch();
  return e;
}

}  // namespace lake
