// mlp_family.cu — NEXT-4: the second workload on the fused-MLP family (include/lake_mlp.h).
// Small classifier MLPs of the kind LAKE ports for load balancing (MLLB, §7.3)
// and readahead classification (KML, §7.4): widths <= 64, 1..4 weight layers,
// ReLU or sigmoid hidden units, identity output, first-max class. Batch scoring =
// score_features (Table 1).
//
// These networks are far too narrow for tensor cores (K = 5..15: an MMA's K is 16, and the
// whole network is ~300-450 FMAs per input), so the kernel is an FP32 CUDA-core kernel
// whose bound is the FP32 pipe (plus the SFU work of sigmoid) with HBM close behind
// (DESIGN.md §6.7):
//  * one thread owns RPT input rows and computes the whole network for them in registers:
//    acc[RPT][MAXW] over the padded output width, k-loop in ascending order, so every
//    output is summed exactly in the oracle's order (ReLU models are bit-exact, R15);
//  * the model image (W^T per layer, [K][Np] with Np = roundup(N, 8), zero-padded, then
//    the bias) is copied into SMEM once per CTA; every thread of a warp reads the same
//    weights, so each LDS.128 is a broadcast feeding 4 * RPT FMAs;
//  * input rows are staged through SMEM by cp.async, double-buffered (the next tile's rows
//    land while this tile computes); odd input widths are read in place, even ones are
//    re-laid at an odd row stride first (conflict-free per-thread reads); hidden activations
//    live in SMEM columns owned by their thread ([MAXW][rows], conflict-free);
//  * persistent grid-stride over 128*RPT-row tiles.
#include <cuda_pipeline.h>
#include <cuda_runtime.h>

#include <cmath>
#include <cstring>
#include <atomic>
#include <mutex>
#include <vector>

#include "../../include/lake_mlp.h"
#include "lake_internal.h"
#include "lake_ptx.cuh"

namespace lake {
namespace {

constexpr int kFamThreads = 128;
// rows per thread of the compile-time-shape kernels for large batches (each weight LDS.128
// then feeds 4 * RPT FMAs); A/B on B200: MLLB 2 -> 4 rows +12%
#ifndef LAKE_FAM_RPT
#define LAKE_FAM_RPT 4
#endif
#ifndef LAKE_FAM_RPT_KML
#define LAKE_FAM_RPT_KML 2
#endif
constexpr int kFamMaxDevices = 64;

struct FamModel {
  const float *img;               // device image (layout above)
  int32_t n_layers;
  int32_t act;
  int32_t widths[LAKE_MLP_MAX_LAYERS + 1];
  int32_t np[LAKE_MLP_MAX_LAYERS + 1];    // padded widths (multiple of 8); np[0] unused
  int32_t off_w[LAKE_MLP_MAX_LAYERS];     // float offsets of W^T_l and b_l in the image
  int32_t off_b[LAKE_MLP_MAX_LAYERS];
  int32_t img_floats;                     // multiple of 4
  int32_t max_np;                         // max over np[1..n_layers]
  const float *img_fx;                    // fixed-shape image (FixedShape layout) or null
  int32_t img_fx_floats;
  int32_t fixed;                          // 0 generic, 1 MLLB shape, 2 KML shape
};

__host__ __device__ constexpr int round8(int x) { return (x + 7) & ~7; }

// acc[i][j] += a_i(k) * W^T[k][j] for k = 0..K-1 in order, j < 8*NCH (the layer's padded
// width). a_i(k) = a[i * kFamThreads * a_rs + k * a_ks]. NCH is a template parameter so
// the k-loop body is branch-free and can be unrolled (loads of k+1.. issued early).
template <int NCH, int RPT, int MAXW>
__device__ __forceinline__ void dense_acc(float (&acc)[RPT][MAXW], const float *a, int a_rs,
                                          int a_ks, const float *wt, int Np, int K) {
#pragma unroll 4
  for (int k = 0; k < K; ++k) {
    float av[RPT];
#pragma unroll
    for (int i = 0; i < RPT; ++i) av[i] = a[i * 128 * a_rs + k * a_ks];  // 128 = kFamThreads
    const float4 *wrow = reinterpret_cast<const float4 *>(wt + k * Np);
#pragma unroll
    for (int jb = 0; jb < NCH; ++jb) {
      const float4 w0 = wrow[2 * jb], w1 = wrow[2 * jb + 1];
      const float w[8] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w};
#pragma unroll
      for (int i = 0; i < RPT; ++i)
#pragma unroll
        for (int e = 0; e < 8; ++e)
          acc[i][jb * 8 + e] = __fmaf_rn(av[i], w[e], acc[i][jb * 8 + e]);
    }
  }
}

template <int RPT, int MAXW>
__device__ __forceinline__ void dense_dispatch(float (&acc)[RPT][MAXW], const float *a, int a_rs,
                                               int a_ks, const float *wt, int Np, int K) {
  switch (Np >> 3) {
    case 1: dense_acc<1, RPT, MAXW>(acc, a, a_rs, a_ks, wt, Np, K); break;
    case 2: dense_acc<2, RPT, MAXW>(acc, a, a_rs, a_ks, wt, Np, K); break;
    default:
      if constexpr (MAXW >= 32) {
        switch (Np >> 3) {
          case 3: dense_acc<3, RPT, MAXW>(acc, a, a_rs, a_ks, wt, Np, K); break;
          case 4: dense_acc<4, RPT, MAXW>(acc, a, a_rs, a_ks, wt, Np, K); break;
          default:
            if constexpr (MAXW >= 64) {
              switch (Np >> 3) {
                case 5: dense_acc<5, RPT, MAXW>(acc, a, a_rs, a_ks, wt, Np, K); break;
                case 6: dense_acc<6, RPT, MAXW>(acc, a, a_rs, a_ks, wt, Np, K); break;
                case 7: dense_acc<7, RPT, MAXW>(acc, a, a_rs, a_ks, wt, Np, K); break;
                default: dense_acc<8, RPT, MAXW>(acc, a, a_rs, a_ks, wt, Np, K); break;
              }
            }
        }
      }
  }
}

#ifndef LAKE_FAM_IEEE_SIGMOID
// sigmoid on the SFU (R27): 2^(-z log2 e) by ex2.approx, then rcp.approx - 3 instructions
// instead of the ~20 of expf + IEEE division; KML-shape throughput x1.8 (A/B), outputs stay
// within the 1e-5 relative parity bound against the oracle's binary32 definition
__device__ __forceinline__ float fam_sigmoid(float z) {
  float e, r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e) : "f"(z * -1.4426950408889634f));
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(1.0f + e));
  return r;
}
#else
__device__ __forceinline__ float fam_sigmoid(float z) {
  return __fdiv_rn(1.0f, __fadd_rn(1.0f, expf(-z)));
}
#endif
__device__ __forceinline__ float fam_act(int act, float z) {
  return act == LAKE_ACT_RELU ? ((z > 0.0f) ? z : 0.0f) : fam_sigmoid(z);
}

// Per-row network evaluation, generic shapes (runtime widths <= MAXW): activations round
// trip through SMEM columns between layers.
template <int MAXW>
struct GenericBody {
  static constexpr bool kFixed = false;
  __host__ __device__ static int sh_floats(int rows) { return MAXW * rows; }
  template <int RPT>
  __device__ static void run(const FamModel &m, const float *sw, const float *sx, int sxs,
                             float *sh, int tid, int64_t row0, int cnt, int32_t *classes,
                             float *out) {
    constexpr int ROWS = kFamThreads * RPT;
    const int L = m.n_layers;
    float acc[RPT][MAXW];
    for (int l = 0; l < L; ++l) {
      const int K = m.widths[l], N = m.widths[l + 1], Np = m.np[l + 1];
      const float *wt = sw + m.off_w[l];
#pragma unroll
      for (int i = 0; i < RPT; ++i)
#pragma unroll
        for (int j = 0; j < MAXW; ++j) acc[i][j] = 0.0f;
      if (l == 0) dense_dispatch<RPT, MAXW>(acc, sx + tid * sxs, sxs, 1, wt, Np, K);
      else dense_dispatch<RPT, MAXW>(acc, sh + tid, 1, ROWS, wt, Np, K);
      const float *b = sw + m.off_b[l];
      if (l + 1 < L) {
#pragma unroll
        for (int j = 0; j < MAXW; ++j) {
          if (j < N) {
            const float bj = b[j];
#pragma unroll
            for (int i = 0; i < RPT; ++i)
              sh[j * ROWS + tid + i * kFamThreads] = fam_act(m.act, __fadd_rn(acc[i][j], bj));
          }
        }
      } else {
#pragma unroll
        for (int i = 0; i < RPT; ++i) {
          const int r = tid + i * kFamThreads;
          if (r >= cnt) continue;
          const int64_t row = row0 + r;
          float best = 0.0f;
          int bi = 0;
#pragma unroll
          for (int j = 0; j < MAXW; ++j) {
            if (j < N) {
              const float z = __fadd_rn(acc[i][j], b[j]);
              if (out) out[row * N + j] = z;
              if (j == 0) best = z;
              else if (z > best) { best = z; bi = j; }  // first max; NaN never wins
            }
          }
          classes[row] = bi;
        }
      }
    }
  }
};

// Fixed shapes (the two readings the bench runs, R25/R26): widths, offsets and activation
// are compile-time, the whole network is unrolled with every activation in registers, the
// weights are read as LDS.128 broadcasts of W[j][k..k+3] (row-major, K padded to 4; the pad
// is never read) and each weight feeds RPT rows. Same operation order as the oracle.
template <int ACT_, int... Ws>
struct FixedShape {
  static constexpr int L = sizeof...(Ws) - 1;
  static constexpr int ACT = ACT_;
  __host__ __device__ static constexpr int w(int i) {
    constexpr int a[] = {Ws...};
    return a[i];
  }
  __host__ __device__ static constexpr int maxw() {
    constexpr int a[] = {Ws...};
    int r = 0;
    for (int i = 0; i <= L; ++i) r = a[i] > r ? a[i] : r;
    return r;
  }
  __host__ __device__ static constexpr int kp(int l) { return (w(l) + 3) & ~3; }
  __host__ __device__ static constexpr int off_w(int l) {
    int o = 0;
    for (int i = 0; i < l; ++i) o += w(i + 1) * kp(i) + ((w(i + 1) + 3) & ~3);
    return o;
  }
  __host__ __device__ static constexpr int off_b(int l) { return off_w(l) + w(l + 1) * kp(l); }
  __host__ __device__ static constexpr int img_floats() { return off_w(L); }
};
using MllbShape = FixedShape<LAKE_ACT_RELU, 15, 10, 10, 2>;
using KmlShape = FixedShape<LAKE_ACT_SIGMOID, 5, 15, 15, 4>;


template <class S, int RPT, int l>
__device__ __forceinline__ void fixed_layers(float (&h)[RPT][S::maxw()], const float *sw,
                                             int tid, int64_t row0, int cnt, int32_t *classes,
                                             float *out) {
  constexpr int K = S::w(l), N = S::w(l + 1), Kp = S::kp(l);
  constexpr int OW = S::off_w(l), OB = S::off_b(l);
  float z[RPT][S::maxw()];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    float acc[RPT];
#pragma unroll
    for (int i = 0; i < RPT; ++i) acc[i] = 0.0f;
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const float wv = sw[OW + j * Kp + k];
#pragma unroll
      for (int i = 0; i < RPT; ++i) acc[i] = __fmaf_rn(h[i][k], wv, acc[i]);
    }
    const float bj = sw[OB + j];
#pragma unroll
    for (int i = 0; i < RPT; ++i) z[i][j] = __fadd_rn(acc[i], bj);
  }
  if constexpr (l + 1 < S::L) {
#pragma unroll
    for (int i = 0; i < RPT; ++i)
#pragma unroll
      for (int j = 0; j < N; ++j) h[i][j] = fam_act(S::ACT, z[i][j]);
    fixed_layers<S, RPT, l + 1>(h, sw, tid, row0, cnt, classes, out);
  } else {
#pragma unroll
    for (int i = 0; i < RPT; ++i) {
      const int r = tid + i * kFamThreads;
      if (r >= cnt) continue;
      const int64_t row = row0 + r;
      float best = z[i][0];
      int bi = 0;
#pragma unroll
      for (int j = 1; j < N; ++j)
        if (z[i][j] > best) { best = z[i][j]; bi = j; }  // first max; NaN never wins
      if (out) {
#pragma unroll
        for (int j = 0; j < N; ++j) out[row * N + j] = z[i][j];
      }
      classes[row] = bi;
    }
  }
}

template <class S>
struct FixedBody {
  static constexpr bool kFixed = true;
  __host__ __device__ static int sh_floats(int) { return 0; }
  template <int RPT>
  __device__ static void run(const FamModel &, const float *sw, const float *sx, int sxs,
                             float *, int tid, int64_t row0, int cnt, int32_t *classes,
                             float *out) {
    float h[RPT][S::maxw()];
#pragma unroll
    for (int i = 0; i < RPT; ++i)
#pragma unroll
      for (int k = 0; k < S::w(0); ++k) h[i][k] = sx[(tid + i * kFamThreads) * sxs + k];
    fixed_layers<S, RPT, 0>(h, sw, tid, row0, cnt, classes, out);
  }
};

// Tile driver shared by both bodies: model image -> SMEM once per CTA, persistent
// grid-stride over ROWS-row tiles, cp.async double-buffered row staging.
template <class Body, int RPT>
__global__ void __launch_bounds__(kFamThreads)
mlp_family_kernel(const float *__restrict__ x, int64_t n, const __grid_constant__ FamModel m,
                  int32_t *__restrict__ classes, float *__restrict__ out) {
  constexpr int ROWS = kFamThreads * RPT;
  extern __shared__ float4 fam_smem4[];
  float *sw = reinterpret_cast<float *>(fam_smem4);
  const float *img = Body::kFixed ? m.img_fx : m.img;
  const int img_floats = Body::kFixed ? m.img_fx_floats : m.img_floats;
  const int W0 = m.widths[0];
  const int W0p = W0 | 1;                      // odd row stride: conflict-free row reads
  const int xbuf = (ROWS * W0 + 3) & ~3;       // floats per staging buffer (16-B multiple)
  float *const sxb0 = sw + img_floats, *const sxb1 = sxb0 + xbuf;
  float *sxp = sxb1 + xbuf;                    // padded copy (even W0 only): [ROWS][W0p]
  // generic body: hidden activations [MAXW][ROWS]; one buffer serves every layer, because
  // a thread only touches its own rows' column and writes layer l's outputs after its
  // k-loop has read all of layer l's inputs
  float *sh = sxp + ((W0 & 1) ? 0 : ROWS * W0p);
  const int tid = threadIdx.x;
  const bool vec = (reinterpret_cast<uintptr_t>(x) & 15) == 0;

  for (int i = tid; i < img_floats / 4; i += kFamThreads)
    fam_smem4[i] = __ldg(reinterpret_cast<const float4 *>(img) + i);

  const int64_t n_tiles = (n + ROWS - 1) / ROWS;
  // One tile's rows are cnt*W0 contiguous floats, and tile * ROWS * W0 * 4 bytes is a
  // multiple of 16: with a 16-byte aligned x, one thread moves the tile with a single bulk
  // copy (TMA engine, completion on an mbarrier) plus at most 3 tail floats; otherwise every
  // thread issues 4-byte cp.async copies.
  __shared__ __align__(8) uint64_t fam_bar[2];
  const uint32_t bar0 = ptx::smem_u32(&fam_bar[0]);
  if (vec && tid == 0) {
    ptx::mbar_init(bar0, 1);
    ptx::mbar_init(bar0 + 8, 1);
    ptx::fence_mbar_init();
  }
  auto stage = [&](int64_t tile, float *dst, uint32_t bar) {
    const int64_t row0 = tile * ROWS;
    const int cnt = (int)((n - row0) < ROWS ? (n - row0) : ROWS);
    const int nf = cnt * W0;
    const float *src = x + row0 * W0;
    if (vec) {
      if (tid == 0) {
        const uint32_t bulk = (uint32_t)(nf & ~3) * 4;
        ptx::mbar_arrive_expect_tx(bar, bulk);
        if (bulk) ptx::bulk_g2s(ptx::smem_u32(dst), src, bulk, bar);
      }
      const int i = (nf & ~3) + tid;  // tail: plain loads, made visible by __syncthreads
      if (i < nf) dst[i] = __ldg(src + i);
    } else {
      for (int i = tid; i < nf; i += kFamThreads)
        __pipeline_memcpy_async(dst + i, src + i, 4);
      __pipeline_commit();
    }
  };
  __syncthreads();  // barrier init visible before the first copy
  if ((int64_t)blockIdx.x < n_tiles) stage(blockIdx.x, sxb0, bar0);

  int it = 0;
  for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
    const int64_t row0 = tile * ROWS;
    const int cnt = (int)((n - row0) < ROWS ? (n - row0) : ROWS);
    __syncthreads();  // image copied; every thread is done with the previous tile's rows
    if (tile + gridDim.x < n_tiles)
      stage(tile + gridDim.x, (it & 1) ? sxb0 : sxb1, bar0 + ((it + 1) & 1) * 8);
    else if (!vec)
      __pipeline_commit();
    if (vec) ptx::mbar_wait(bar0 + (it & 1) * 8, (uint32_t)((it >> 1) & 1));
    else __pipeline_wait_prior(1);  // this thread's copies of the current tile have landed
    __syncthreads();                // ... and everyone's
    const float *sx = (it & 1) ? sxb1 : sxb0;
    int sxs = W0;
    if (!(W0 & 1)) {  // even width: re-lay rows at an odd stride (bank-conflict-free reads)
      for (int i = tid; i < cnt * W0; i += kFamThreads) {
        const int r = i / W0, k = i - r * W0;
        sxp[r * W0p + k] = sx[i];
      }
      __syncthreads();
      sx = sxp;
      sxs = W0p;
    }
    Body::template run<RPT>(m, sw, sx, sxs, sh, tid, row0, cnt, classes, out);
  }
}

// ------------------------------------------------------------------ registry + C ABI
struct FamSlot {
  bool loaded = false;
  FamModel m{};
  float *dimg = nullptr;
};
struct FamDevice {
  FamSlot slot[LAKE_MLP_MAX_MODELS];
};
std::mutex g_fam_mu;
// test hook: route the fixed shapes through the generic kernel (lake_mlp_set_generic)
bool g_fam_force_generic = false;
FamDevice *g_fam[kFamMaxDevices] = {};

int fam_cuda_status(cudaError_t e) {
  if (e == cudaSuccess) return LAKE_OK;
  if (e == cudaErrorMemoryAllocation) return LAKE_ERR_NOMEM;
  return LAKE_ERR_CUDA;
}

struct FamDeviceGuard {
  int prev = -1;
  bool ok = true;
  explicit FamDeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) { ok = false; return; }
    if (prev != dev && cudaSetDevice(dev) != cudaSuccess) ok = false;
  }
  ~FamDeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

bool valid_shape(int32_t n_layers, const int32_t *widths) {
  if (!widths || n_layers < 1 || n_layers > LAKE_MLP_MAX_LAYERS) return false;
  for (int l = 0; l <= n_layers; ++l)
    if (widths[l] < 1 || widths[l] > LAKE_MLP_MAX_WIDTH) return false;
  return widths[n_layers] >= 2;
}

template <class Body>
size_t fam_smem_bytes(const FamModel &m, int rpt) {
  const int rows = kFamThreads * rpt;
  const int w0 = m.widths[0];
  const size_t xbuf = (size_t)((rows * w0 + 3) & ~3);
  const size_t img = Body::kFixed ? (size_t)m.img_fx_floats : (size_t)m.img_floats;
  return (img + 2 * xbuf + ((w0 & 1) ? 0 : (size_t)rows * (w0 | 1)) +
          (size_t)Body::sh_floats(rows)) * 4;
}

template <class Body, int RPT>
cudaError_t fam_launch(const float *x, int64_t n, const FamModel &m, int32_t *cls, float *out,
                       cudaStream_t s, int sms) {
  const size_t smem = fam_smem_bytes<Body>(m, RPT);
  // per-device caches shared by host threads: atomics (a race only repeats a query)
  static std::atomic<bool> attr_set[kFamMaxDevices];
  int dev = 0;
  cudaGetDevice(&dev);
  dev &= kFamMaxDevices - 1;
  if (!attr_set[dev].load(std::memory_order_acquire)) {
    cudaError_t e = cudaFuncSetAttribute(mlp_family_kernel<Body, RPT>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, 226 * 1024);  // + static barriers
    if (e != cudaSuccess) return e;
    attr_set[dev].store(true, std::memory_order_release);
  }
  // resident CTAs per SM for this SMEM size (cached: the query costs microseconds)
  static std::atomic<int> occ_cache[kFamMaxDevices][64];
  const int key = (int)((smem + 4095) / 4096) & 63;
  int per_sm = occ_cache[dev][key].load(std::memory_order_relaxed);
  if (!per_sm) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessorWithFlags(&per_sm, mlp_family_kernel<Body, RPT>,
                                                           kFamThreads, key * 4096, 0);
    if (per_sm < 1) per_sm = 1;
    occ_cache[dev][key].store(per_sm, std::memory_order_relaxed);
  }
  const int64_t rows = (int64_t)kFamThreads * RPT;
  const int64_t tiles = (n + rows - 1) / rows;
  const int64_t cap = (int64_t)sms * per_sm;
  const int grid = (int)(tiles < cap ? tiles : cap);
  mlp_family_kernel<Body, RPT><<<grid, kFamThreads, smem, s>>>(x, n, m, cls, out);
  return cudaGetLastError();
}

template <class S>
bool shape_is(const FamModel &m) {
  if (m.n_layers != S::L || m.act != S::ACT) return false;
  for (int l = 0; l <= S::L; ++l)
    if (m.widths[l] != S::w(l)) return false;
  return true;
}

template <class S>
void build_fixed_image(const float *blob, std::vector<float> &img) {
  img.assign((size_t)S::img_floats(), 0.0f);
  const float *q = blob;
  for (int l = 0; l < S::L; ++l) {
    const int K = S::w(l), N = S::w(l + 1);
    for (int j = 0; j < N; ++j)
      for (int k = 0; k < K; ++k) img[(size_t)S::off_w(l) + (size_t)j * S::kp(l) + k] = q[j * K + k];
    q += N * K;
    for (int j = 0; j < N; ++j) img[(size_t)S::off_b(l) + j] = q[j];
    q += N;
  }
}

}  // namespace

}  // namespace lake

using namespace lake;

extern "C" {

size_t lake_mlp_blob_floats(int32_t n_layers, const int32_t *widths) {
  if (!valid_shape(n_layers, widths)) return 0;
  size_t t = 0;
  for (int l = 0; l < n_layers; ++l) t += (size_t)widths[l + 1] * widths[l] + widths[l + 1];
  return t;
}

static int mlp_load_impl(int32_t model_id, int32_t n_layers, const int32_t *widths, int32_t act,
                  const float *blob, size_t n_floats, int32_t device) {
  if (model_id < 0 || model_id >= LAKE_MLP_MAX_MODELS) return LAKE_ERR_INVAL;
  if (!valid_shape(n_layers, widths)) return LAKE_ERR_INVAL;
  if (act != LAKE_ACT_RELU && act != LAKE_ACT_SIGMOID) return LAKE_ERR_INVAL;
  if (!blob || n_floats != lake_mlp_blob_floats(n_layers, widths)) return LAKE_ERR_INVAL;
  if (device < 0 || device >= kFamMaxDevices) return LAKE_ERR_INVAL;
  for (size_t i = 0; i < n_floats; ++i)
    if (!std::isfinite(blob[i])) return LAKE_ERR_INVAL;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess) return LAKE_ERR_CUDA;
  if (device >= ndev) return LAKE_ERR_INVAL;

  // image: per layer W^T [K][Np] (zero-padded columns), then b [Np]
  FamModel m;
  std::memset(&m, 0, sizeof(m));
  m.n_layers = n_layers;
  m.act = act;
  int p = 0;
  for (int l = 0; l <= n_layers; ++l) m.widths[l] = widths[l];
  for (int l = 0; l < n_layers; ++l) {
    const int K = widths[l], Np = round8(widths[l + 1]);
    m.np[l + 1] = Np;
    if (Np > m.max_np) m.max_np = Np;
    m.off_w[l] = p;
    p += K * Np;
    m.off_b[l] = p;
    p += Np;
  }
  m.img_floats = (p + 3) & ~3;
  std::vector<float> img((size_t)m.img_floats, 0.0f);
  const float *q = blob;
  for (int l = 0; l < n_layers; ++l) {
    const int K = widths[l], N = widths[l + 1], Np = m.np[l + 1];
    for (int j = 0; j < N; ++j)
      for (int k = 0; k < K; ++k) img[(size_t)m.off_w[l] + (size_t)k * Np + j] = q[(size_t)j * K + k];
    q += (size_t)N * K;
    for (int j = 0; j < N; ++j) img[(size_t)m.off_b[l] + j] = q[j];
    q += N;
  }

  // compile-time-shape image for the two shapes with a specialised kernel (R25/R26)
  std::vector<float> fx;
  if (shape_is<MllbShape>(m)) {
    m.fixed = 1;
    build_fixed_image<MllbShape>(blob, fx);
  } else if (shape_is<KmlShape>(m)) {
    m.fixed = 2;
    build_fixed_image<KmlShape>(blob, fx);
  }
  m.img_fx_floats = (int32_t)fx.size();
  const size_t total = img.size() + fx.size();

  std::lock_guard<std::mutex> lk(g_fam_mu);
  FamDeviceGuard dg(device);
  if (!dg.ok) return LAKE_ERR_CUDA;
  if (!g_fam[device]) g_fam[device] = new (std::nothrow) FamDevice();
  if (!g_fam[device]) return LAKE_ERR_NOMEM;
  float *d = nullptr;
  if (cudaMalloc(&d, total * 4) != cudaSuccess) return LAKE_ERR_NOMEM;
  if (cudaMemcpy(d, img.data(), img.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
      (!fx.empty() && cudaMemcpy(d + img.size(), fx.data(), fx.size() * 4,
                                 cudaMemcpyHostToDevice) != cudaSuccess)) {
    release_device(d, device);
    return LAKE_ERR_CUDA;
  }
  m.img_fx = fx.empty() ? nullptr : d + img.size();
  FamSlot &s = g_fam[device]->slot[model_id];
  release_device(s.dimg, device);  // deferred while a persistent server runs
  m.img = d;
  s.m = m;
  s.dimg = d;
  s.loaded = true;
  return LAKE_OK;
}

int lake_mlp_load(int32_t model_id, int32_t n_layers, const int32_t *widths, int32_t act,
                  const float *blob, size_t n_floats, int32_t device) {
  // the image building allocates host vectors: never let bad_alloc cross the C ABI
  try {
    return mlp_load_impl(model_id, n_layers, widths, act, blob, n_floats, device);
  } catch (...) {
    return LAKE_ERR_NOMEM;
  }
}

int lake_mlp_unload(int32_t model_id, int32_t device) {
  if (model_id < 0 || model_id >= LAKE_MLP_MAX_MODELS) return LAKE_ERR_INVAL;
  if (device < 0 || device >= kFamMaxDevices) return LAKE_ERR_INVAL;
  std::lock_guard<std::mutex> lk(g_fam_mu);
  if (!g_fam[device] || !g_fam[device]->slot[model_id].loaded) return LAKE_ERR_NOMODEL;
  FamDeviceGuard dg(device);
  if (!dg.ok) return LAKE_ERR_CUDA;
  FamSlot &s = g_fam[device]->slot[model_id];
  release_device(s.dimg, device);  // deferred while a persistent server runs
  s = FamSlot();
  return LAKE_OK;
}

size_t lake_mlp_host_staging_bytes(int64_t n, int32_t width_in, int32_t classes) {
  if (n < 0 || width_in < 1 || width_in > LAKE_MLP_MAX_WIDTH || classes < 2 ||
      classes > LAKE_MLP_MAX_WIDTH)
    return 0;
  const size_t r = (size_t)(n > 0 ? n : 1);
  auto a256 = [](size_t x) { return (x + 255) & ~(size_t)255; };
  return a256(r * width_in * 4) + a256(r * 4) + a256(r * classes * 4);
}

int lake_mlp_infer_host(const float *h_x, int64_t n, int32_t model_id, int32_t *h_classes,
                        float *h_out, void *d_staging, size_t staging_bytes, void *stream) {
  if (n < 0 || n > (int64_t)INT32_MAX) return LAKE_ERR_INVAL;
  if (n == 0) return LAKE_OK;
  if (!h_x || !h_classes) return LAKE_ERR_INVAL;
  if (model_id < 0 || model_id >= LAKE_MLP_MAX_MODELS) return LAKE_ERR_NOMODEL;
  int device = 0;
  if (cudaGetDevice(&device) != cudaSuccess) return LAKE_ERR_CUDA;
  if (device < 0 || device >= kFamMaxDevices) return LAKE_ERR_NOMODEL;
  int32_t w0, C;
  {
    std::lock_guard<std::mutex> lk(g_fam_mu);
    if (!g_fam[device] || !g_fam[device]->slot[model_id].loaded) return LAKE_ERR_NOMODEL;
    const FamModel &m = g_fam[device]->slot[model_id].m;
    w0 = m.widths[0];
    C = m.widths[m.n_layers];
  }
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  // zero-copy when every host buffer is pinned and mapped
  auto mapped = [](const void *h) -> void * {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, h) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    return (a.type == cudaMemoryTypeHost) ? a.devicePointer : nullptr;
  };
  void *dx = mapped(h_x), *dc = mapped(h_classes), *dout = h_out ? mapped(h_out) : nullptr;
  int rc;
  if (dx && dc && (!h_out || dout)) {
    rc = lake_mlp_infer(static_cast<const float *>(dx), n, model_id, static_cast<int32_t *>(dc),
                        static_cast<float *>(dout), stream);
    if (rc != LAKE_OK) return rc;
    return fam_cuda_status(cudaStreamSynchronize(s));
  }
  if (!d_staging || staging_bytes < lake_mlp_host_staging_bytes(n, w0, C)) return LAKE_ERR_NOMEM;
  auto a256 = [](size_t x) { return (x + 255) & ~(size_t)255; };
  uint8_t *b = static_cast<uint8_t *>(d_staging);
  float *sx = reinterpret_cast<float *>(b);
  int32_t *sc = reinterpret_cast<int32_t *>(b + a256((size_t)n * w0 * 4));
  float *so = reinterpret_cast<float *>(b + a256((size_t)n * w0 * 4) + a256((size_t)n * 4));
  cudaError_t e = cudaMemcpyAsync(sx, h_x, (size_t)n * w0 * 4, cudaMemcpyHostToDevice, s);
  if (e != cudaSuccess) return fam_cuda_status(e);
  rc = lake_mlp_infer(sx, n, model_id, sc, h_out ? so : nullptr, stream);
  if (rc != LAKE_OK) return rc;
  e = cudaMemcpyAsync(h_classes, sc, (size_t)n * 4, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess && h_out)
    e = cudaMemcpyAsync(h_out, so, (size_t)n * C * 4, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  return fam_cuda_status(e);
}

int lake_mlp_force_generic(int32_t enable) {
  std::lock_guard<std::mutex> lk(g_fam_mu);
  const int prev = g_fam_force_generic ? 1 : 0;
  g_fam_force_generic = enable != 0;
  return prev;
}

int lake_mlp_model_shape(int32_t model_id, int32_t device, int32_t *n_layers_out,
                         int32_t *widths_out, int32_t *act_out) {
  if (!n_layers_out || !widths_out || !act_out) return LAKE_ERR_INVAL;
  if (model_id < 0 || model_id >= LAKE_MLP_MAX_MODELS) return LAKE_ERR_NOMODEL;
  if (device < 0 || device >= kFamMaxDevices) return LAKE_ERR_INVAL;
  std::lock_guard<std::mutex> lk(g_fam_mu);
  if (!g_fam[device] || !g_fam[device]->slot[model_id].loaded) return LAKE_ERR_NOMODEL;
  const FamModel &m = g_fam[device]->slot[model_id].m;
  *n_layers_out = m.n_layers;
  for (int l = 0; l <= m.n_layers; ++l) widths_out[l] = m.widths[l];
  *act_out = m.act;
  return LAKE_OK;
}

int lake_mlp_infer(const float *x, int64_t n, int32_t model_id, int32_t *classes, float *out,
                   void *stream) {
  if (n < 0 || n > (int64_t)INT32_MAX) return LAKE_ERR_INVAL;
  if (n == 0) return LAKE_OK;
  if (!x || !classes) return LAKE_ERR_INVAL;
  if ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(classes) |
       reinterpret_cast<uintptr_t>(out)) & 3)
    return LAKE_ERR_INVAL;
  if (model_id < 0 || model_id >= LAKE_MLP_MAX_MODELS) return LAKE_ERR_NOMODEL;
  int device = 0;
  if (cudaGetDevice(&device) != cudaSuccess) return LAKE_ERR_CUDA;
  if (device < 0 || device >= kFamMaxDevices) return LAKE_ERR_NOMODEL;
  FamModel m;
  {
    std::lock_guard<std::mutex> lk(g_fam_mu);
    if (!g_fam[device] || !g_fam[device]->slot[model_id].loaded) return LAKE_ERR_NOMODEL;
    m = g_fam[device]->slot[model_id].m;
  }
  static std::atomic<int> sms_cache[kFamMaxDevices];
  int sms = sms_cache[device].load(std::memory_order_relaxed);
  if (!sms) {
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess)
      return LAKE_ERR_CUDA;
    sms_cache[device].store(sms, std::memory_order_relaxed);
  }
  // width class of the register tile; two rows per thread once the batch fills the GPU
  const int maxw = m.max_np <= 16 ? 16 : m.max_np <= 32 ? 32 : 64;
  const bool big = n > (int64_t)kFamThreads * sms * 2;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  cudaError_t e;
  bool generic;
  {
    std::lock_guard<std::mutex> lk(g_fam_mu);
    generic = g_fam_force_generic;
  }
  if (m.fixed == 1 && !generic)
    e = big ? fam_launch<FixedBody<MllbShape>, LAKE_FAM_RPT>(x, n, m, classes, out, s, sms)
            : fam_launch<FixedBody<MllbShape>, 1>(x, n, m, classes, out, s, sms);
  else if (m.fixed == 2 && !generic)
    e = big ? fam_launch<FixedBody<KmlShape>, LAKE_FAM_RPT_KML>(x, n, m, classes, out, s, sms)
            : fam_launch<FixedBody<KmlShape>, 1>(x, n, m, classes, out, s, sms);
  else if (maxw == 16)
    e = big ? fam_launch<GenericBody<16>, 2>(x, n, m, classes, out, s, sms)
            : fam_launch<GenericBody<16>, 1>(x, n, m, classes, out, s, sms);
  else if (maxw == 32)
    e = big ? fam_launch<GenericBody<32>, 2>(x, n, m, classes, out, s, sms)
            : fam_launch<GenericBody<32>, 1>(x, n, m, classes, out, s, sms);
  else
    e = fam_launch<GenericBody<64>, 1>(x, n, m, classes, out, s, sms);
  count_launch();
  return fam_cuda_status(e);
}

}  // extern "C"
