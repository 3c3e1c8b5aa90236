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
//  * Warp roles (20 warps): w0-1 digitisers (raw records -> fp16 digits, double-buffered
//    X), w2 weight loader + TMEM allocator, w19 MMA issuer (leader CTA, one thread),
//    w3-18 epilogue, 4 per TMEM lane quadrant, 16 columns of each 64-column chunk each (tcgen05.ld -> +bias -> ReLU -> fp16 -> st.shared -> mbarrier; the last
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

#include <atomic>
#include <cstdlib>

#include "digitize.cuh"
#include "lake_internal.h"
#include "lake_ptx.cuh"

// ---- optional timeline trace (make trace): clock64 stamps from the leader CTA of cluster 0
#ifdef LAKE_TRACE
// per-stream event logs: stream 0 MMA thread, 1 epilogue warp 4, 2 epilogue warp 11,
// 3 digitiser; thread-local write index (no atomics), 2 u64 per event, 64K events each
__device__ unsigned long long *g_lake_trace = nullptr;
#ifdef LAKE_TRACE_SMEM
// low-overhead variant: events of tiles [LAKE_TRACE_TW0, +3) go to a 32-KB SMEM log after the
// kernel's layout (st.shared, no global traffic) and are copied to g_lake_trace at exit;
// 512 events per stream, fp16/bf16 only (tf32 has no SMEM to spare)
#ifndef LAKE_TRACE_TW0
#define LAKE_TRACE_TW0 200
#endif
#define LAKE_TRACE_CAP 512u
#define LAKE_TEV(kind, tile, layer, chunk)                                                   \
  do {                                                                                    \
    if (tr_stream >= 0 && (tile) >= LAKE_TRACE_TW0 && (tile) < LAKE_TRACE_TW0 + 3 &&       \
        tr_i < LAKE_TRACE_CAP) {                                                          \
      const unsigned long long k_ = ((unsigned long long)(kind) << 56) |                   \
          ((unsigned long long)(tile) << 24) | ((unsigned long long)(layer) << 8) |        \
          (unsigned long long)(chunk);                                                    \
      const unsigned long long c_ = clock64();                                            \
      asm volatile("st.shared.v2.u64 [%0], {%1, %2};" ::                                   \
                   "r"(tr_smem + 16u * (tr_stream * LAKE_TRACE_CAP + tr_i++)), "l"(k_),      \
                   "l"(c_) : "memory");                                                    \
    }                                                                                     \
  } while (0)
#else
#define LAKE_TRACE_CAP (1u << 16)
#define LAKE_TEV(kind, tile, layer, chunk)                                                   \
  do {                                                                                    \
    if (tr_stream >= 0 && tr_i < LAKE_TRACE_CAP) {                                        \
      unsigned long long *p_ = tr_buf + 2ull * (tr_stream * LAKE_TRACE_CAP + tr_i++);        \
      p_[0] = ((unsigned long long)(kind) << 56) | ((unsigned long long)(tile) << 24) |     \
              ((unsigned long long)(layer) << 8) | (unsigned long long)(chunk);              \
      p_[1] = clock64();                                                                  \
    }                                                                                     \
  } while (0)
#endif
#else
#define LAKE_TEV(kind, tile, layer, chunk) do {} while (0)
#endif
enum TraceKind { T_XFULL = 1, T_TEMPTY = 2, T_HREADY = 3, T_COMMIT = 4, T_DFULL = 5,
                 T_CHUNK = 6, T_LAYER_END = 7, T_XEMPTY = 8, T_XARRIVE = 9, T_ISSUED = 10,
                 T_LDWAIT = 11, T_STS = 12, T_FENCE = 13, T_TOP = 14, T_SCHED = 15,
                 T_WREADY = 16, T_MMA0 = 17, T_CX = 18, T_OHDONE = 19, T_OCOMMIT = 20,
                 T_EHDONE = 21, T_EDOUT = 22, T_ETEMPTY = 23 };

// H (the next layer's A operand) stays in tensor memory, packed in place into the
// accumulator it came from (default); -DLAKE_H_SMEM restores the SMEM H tile + proxy fences.
#ifndef LAKE_H_SMEM
#define LAKE_H_TMEM 1
#endif

namespace lake {
namespace {

#ifndef LAKE_EPI_PER_Q
#define LAKE_EPI_PER_Q 2
#endif
constexpr uint32_t kEpiPerQ = LAKE_EPI_PER_Q;      // epilogue warps per group and quadrant
// Epilogue groups: with 2, one group converts the H-producing layers (0..nh-2) and the
// other the last layer (-> logits), so tile t's logits overlap tile t+1's first epilogues.
#ifndef LAKE_EPI_GROUPS
#define LAKE_EPI_GROUPS 2
#endif
constexpr uint32_t kEpiGroups = LAKE_EPI_GROUPS;
// A/B switch (fp16/bf16, NN+1/NN+2): the last hidden layer as two N = 128 halves, each
// committed on its own barrier, so the logits epilogue starts on columns 0..127 while the
// tensor core computes 128..255. With cta_group::2 an N = 128 MMA takes 64 B rows from each
// CTA, so half h covers features {64h..64h+63} (CTA 0's rows) and {128+64h..} (CTA 1's):
// accumulator column c holds feature nsplit_feature(c), and W_out is staged in that order.
#ifndef LAKE_L2_NSPLIT
#define LAKE_L2_NSPLIT 0
#endif
constexpr bool kL2Split = LAKE_L2_NSPLIT != 0;
__host__ __device__ constexpr uint32_t nsplit_feature(uint32_t c) {
  return c < 64 ? c : c < 128 ? c + 64 : c < 192 ? c - 64 : c;
}
constexpr uint32_t kGroupWarps = 4 * kEpiPerQ;     // warps per epilogue group
constexpr uint32_t kEpiWarps = kEpiGroups * kGroupWarps;
#ifndef LAKE_CHUNKS
#define LAKE_CHUNKS 8
#endif
#ifndef LAKE_EPI_UNROLL  // unroll factor of the epilogue chunk loops (even: register buffers)
#define LAKE_EPI_UNROLL 8
#endif
constexpr int kEpiUnroll = LAKE_EPI_UNROLL;
constexpr uint32_t kChunks = LAKE_CHUNKS;          // H column chunks per layer (MMA K-chunks)
constexpr uint32_t kChunkCols = kHidden / kChunks;
#ifdef LAKE_EPI_INTERLEAVE
// warp hh of a quadrant converts chunks hh, hh+kEpiPerQ, ... (all columns of each), so
// consecutive chunks are produced concurrently by different warps
constexpr bool kInterleave = true;
constexpr uint32_t kEpiCols = kChunkCols;              // columns per warp per chunk
constexpr uint32_t kWarpChunks = kChunks / kEpiPerQ;   // chunks per warp per layer
constexpr uint32_t kHreadyCount = 2 * 4;               // one warp per quadrant, both CTAs
#else
// the kEpiPerQ warps of a quadrant split every chunk's columns between them
constexpr bool kInterleave = false;
constexpr uint32_t kEpiCols = kChunkCols / kEpiPerQ;
constexpr uint32_t kWarpChunks = kChunks;
// H chunk ready (HREADY): the leader CTA's H-group warps arrive through the CTA-local address,
// the peer CTA's group once per chunk after a named barrier (one remote arrive instead of
// eight: C5 fused kernel 3.30 -> 3.28 ms); LAKE_HREADY_PER_WARP restores one remote arrive per
// warp. (The same aggregation for the accumulator releases, TEMPTY, was 1.6% slower.)
#ifndef LAKE_HREADY_PER_WARP
#define LAKE_HREADY_AGG 1
#endif
#ifdef LAKE_HREADY_AGG
constexpr uint32_t kHreadyCount = kGroupWarps + 1;     // leader CTA's H-group warps + the peer
#else
constexpr uint32_t kHreadyCount = 2 * kGroupWarps;     // the H group's warps, both CTAs
#endif
#endif
// MMA K per instruction: 16 (fp16/bf16) or 8 (tf32); K-steps per H chunk
__host__ __device__ constexpr uint32_t kmma(int prec) { return prec == 2 ? 8u : 16u; }
__host__ __device__ constexpr uint32_t ksteps_per_chunk(int prec) { return kChunkCols / kmma(prec); }
constexpr int kThreads = 32 * (3 + kEpiWarps + 1);  // digitisers(2) + loader + epi + MMA
#ifdef LAKE_H_TMEM
constexpr uint32_t kHBytes = 0;                   // H lives in TMEM
#else
constexpr uint32_t kHBytes = 128 * kHidden * 2;   // 64 KB SMEM H tile
#endif
__host__ __device__ constexpr uint32_t x_bytes(int prec) {  // one X tile, 128 rows x 32
  return 128u * kTcK0 * tc_elem_bytes(prec);                // 8 KB / 16 KB (tf32)
}
constexpr uint32_t kLboR128 = 128 * 16;           // K-direction core stride, 128-row operand
constexpr uint32_t kPrmFloats = kHidden + 2 * kHidden + 4;  // last-layer bias | W_out | b_out
constexpr uint32_t kPrm2Words = (kMaxHiddenLayers - 1) * kHidden;  // fp32 H-layer biases
constexpr uint32_t kRedBytes = (kEpiPerQ - 1) * 128 * 2 * 4;  // output-layer partial sums

__host__ __device__ constexpr uint32_t align1k(uint32_t x) { return (x + 1023u) & ~1023u; }

__host__ __device__ constexpr bool streams_w2(int nh, int prec) {
  return tc_resident_bytes(nh, prec) < tc_image_bytes(nh, prec);
}

// input staging (digitisers): two buffers of 128 rows; tf32 only has room for packed rows
__host__ __device__ constexpr uint32_t kStageBytes(int prec) { return prec == 2 ? 2048u : 4608u; }

struct Layout {
  uint32_t ring, h, x, stage, t100, ones, prm, red, prm0, red0, wout, bar, total;
};
// NN kernels (layout 1) with fp16/bf16 operands (out_on_tc): the 2-wide output layer runs on
// the tensor cores. The draining epilogue group packs ReLU(H) in place into the accumulator
// (as for a hidden layer), the MMA issuer multiplies it (A from TMEM) by W_out (N = 16, rows
// 2..15 zero) into the accumulator's last 16 columns, and the group reads back two of them.
// To free those 16 columns the last K-step's packed H goes into the unused half of K-step 13's
// (same warp, earlier chunk: program order makes the overwrite safe). NN tiles were bound by
// the epilogue's CUDA-core work (ReLU + 512 FMAs per row); this leaves 128 packed conversions
// per row. (An SMEM A tile was 3x slower: N=16 SS MMAs ran at ~90 cycles each.) Every
// fp16/bf16 NN tile runs in such a kernel (multi-model calls that mix NN with NN+1/NN+2 run
// one kernel per class, api.cu), so an NN tile gives the same bits in a single-model call and
// inside any multi-model call, and the NN+1/NN+2 kernels carry none of this code.
#ifndef LAKE_NO_OTC
__host__ __device__ constexpr bool out_on_tc(int nh_layout, int prec) {
  // (the in-place packing layout below assumes the default chunking: 8 chunks, 2 warps per
  // quadrant; A/B builds with other chunkings run NN's output layer on the CUDA cores)
  return kEpiGroups == 2 && kEpiPerQ == 2 && kChunks == 8 && nh_layout == 1 && prec != 2;
}
#else  // A/B switch: output layer on CUDA cores for NN too
__host__ __device__ constexpr bool out_on_tc(int, int) { return false; }
#endif
constexpr uint32_t kWoutBytes = 8u * kHidden * 2;    // one group's W_out block (8 rows x K 256)
constexpr uint32_t kLboR8 = 8 * 16;                  // K-direction core stride, 8-row operand
constexpr uint32_t kOutDCol = kHidden - 16;          // output accumulator: columns 240..255
constexpr uint32_t kOutLastA = 13 * 16 + 8;          // last K-step's packed H: K-step 13's gap
// Split of the NN output layer's K = 256 between the tensor cores and the CUDA cores: K-steps
// [0, kOtcKs) (features 0 .. 16 kOtcKs - 1, chunks j < kOtcKs / 2) are packed and multiplied
// by N = 16 MMAs; the rest are ReLU'd and dotted with W_out in fp32 by the draining group
// while it would otherwise wait for those MMAs. A narrow MMA costs >= 62 cycles whatever its
// N (scripts/microbench/umma_dep.cu: per instruction, not an accumulator dependency), so with
// all 16 K-steps on the tensor cores the output layer (~1.3k tensor cycles per tile under
// load) bound the NN kernel.
#ifndef LAKE_OTC_KSTEPS
#define LAKE_OTC_KSTEPS 16
#endif
constexpr uint32_t kOtcKs = LAKE_OTC_KSTEPS;
static_assert(kOtcKs >= 4 && kOtcKs <= 16 && kOtcKs % 2 == 0, "whole chunks on the tensor cores");
// With a CUDA-core share (kOtcKs < 16) the group packs the tensor chunks, arrives on HDONE
// and then does the CUDA chunks while the output MMAs run; those chunks' columns are still
// fp32 H, so the output accumulator moves to columns 24..39, freed by packing chunks 0 and 1
// "shifted": the first warp of the quadrant packs its 16 columns into its own second half
// (32j + 8), the second into its own first half (32j + 16), leaving 32j+24 .. 32j+40 free.
constexpr uint32_t kOtcDCol = kOtcKs == 16 ? kOutDCol : 24u;
__host__ __device__ constexpr uint32_t otc_a_col(uint32_t ks) {
  return kOtcKs == 16 ? (ks + 1 == kHidden / 16 ? kOutLastA : ks * 16)
                      : (ks < 4 && (ks & 1) == 0 ? ks * 16 + 8 : ks * 16);
}
__host__ __device__ constexpr uint32_t otc_wout(int prec) { return tc_w0_half_bytes(prec); }
__host__ __device__ constexpr uint32_t otc_end(int prec) { return otc_wout(prec) + 2 * kWoutBytes; }

__host__ __device__ constexpr Layout tc_layout(int nh_layout, int prec) {
  Layout L{};
  // NN layout with the output layer on the tensor cores: the W_out blocks after W0
  const uint32_t region = out_on_tc(nh_layout, prec) ? otc_end(prec)
                                                      : tc_resident_bytes(nh_layout, prec);
  L.ring = align1k(region);
  L.h = L.ring + (streams_w2(nh_layout, prec) ? kTcRingSlots * kTcRingSlotBytes : 0u);
  L.x = L.h + kHBytes;
  L.stage = L.x + 2 * x_bytes(prec);
  L.t100 = L.stage + 2 * kStageBytes(prec);  // 100 digit pairs (x/10, x%10), operand type
  L.ones = L.t100 + 100 * (prec == 2 ? 8u : 4u);  // "ones" A tile of the bias MMA (fp16/bf16)
  L.prm = L.ones + tc_bias_block_bytes(prec);
  L.red = L.prm + kPrmFloats * 4 + kPrm2Words * 4;
  // group 0's own copy of the output-layer parameters and partial sums: with two epilogue
  // groups, NN tiles (a single layer) are drained by the group of their accumulator buffer
  L.prm0 = L.red + kRedBytes;
  L.red0 = L.prm0 + (kEpiGroups == 2 ? kPrmFloats * 4 : 0u);  // (one group: no private copy)
  L.wout = otc_wout(prec);  // behind W0 in the weight region (out_on_tc layouts only)
  L.bar = L.red0 + (kEpiGroups == 2 ? kRedBytes : 0u);
  L.total = L.bar + 512;
  return L;
}
static_assert(tc_layout(3, 2).total <= 232448, "tf32 NN+2 layout exceeds 227 KB");
static_assert(tc_layout(3, 0).total <= 232448, "fp16 NN+2 layout exceeds 227 KB");

// barrier slots (8 bytes each) inside the barrier block
enum : uint32_t {
  B_WLOAD = 0, B_WREADY = 1, B_XFULL = 2, B_XEMPTY = 4, B_DFULL = 6, B_DFULLX = 8,
  B_TEMPTY = 10, B_HREADY = 12, B_WFREE = 12 + kChunks,
  B_RFULL = 13 + kChunks,                 // [kTcRingSlots] W2 ring slot loaded (tf32 NN+2)
  B_REMPTY = B_RFULL + kTcRingSlots,      // [kTcRingSlots] W2 ring slot consumed
  B_SFULL = B_REMPTY + kTcRingSlots,     // [2] input staging buffer loaded (bulk copy)
  B_HDONE = B_SFULL + 2,                  // [2] out_on_tc: H of buffer b packed (both CTAs)
  B_DOUT = B_HDONE + 2,                   // [2] out_on_tc: output MMA of buffer b done
  B_DHALF = B_DOUT + 2,                   // [2] LAKE_L2_NSPLIT: last layer's first half done
  B_COUNT = B_DHALF + 2
};
constexpr uint32_t kTmemSlot = B_COUNT * 8;  // u32 TMEM base address
static_assert(kTmemSlot + 4 <= 512, "barrier block");

// Per-tile schedule entry. Each role loads tile t+1's entry at the top of tile t (the
// global loads then overlap tile t's work instead of stalling the next iteration).
struct TileInfo {
  const DevModel *model;
  const uint8_t *img;  // this model's weight image for the precision in use
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
  // a model loaded after the host sized the layout (racing the call) is clamped to it: wrong
  // logits for that model, but every role agrees and nothing outside the layout is touched
  ti.nh = ti.model->nh < ts.nh_cap ? ti.model->nh : ts.nh_cap;
  return ti;
}

// Warp roles. The scheduler arbitrates highest-warp-id first, so the latency-critical MMA
// issuer takes the top warp and the epilogue the next eight; the digitisers and the loader
// (off the critical path) sit below.
#ifndef LAKE_MMA_WARP_LOW
constexpr uint32_t kWarpDig = 0;    // warps 0-1: digitisers (64 threads)
constexpr uint32_t kWarpLoad = 2;   // weight loader + TMEM allocator
constexpr uint32_t kWarpEpi = 3;    // epilogue warps (kEpiPerQ per TMEM quadrant)
constexpr uint32_t kWarpMma = kWarpEpi + kEpiWarps;  // MMA issuer (leader CTA, one thread)
#else
constexpr uint32_t kWarpMma = 0;
constexpr uint32_t kWarpDig = 1;
constexpr uint32_t kWarpLoad = 3;
constexpr uint32_t kWarpEpi = 4;
#endif
// A/B switch for the NN kernels with the output layer on the tensor cores (traces show their
// MMA issuer waiting on XFULL): kOtcDigWarps digitiser warps (1 row per thread with 4), the
// extra ones above the MMA warp (warps kThreads / 32 ..), or all of them there with
// LAKE_OTC_DIG_TOP (warps 0-1 then idle), where the scheduler's highest-id-first arbitration
// serves them before the epilogue. Measured slower (C4 NN pre-split 0.2418 ms with 2 warps
// at 0-1; 4 at the top 0.2556, 2 at the top 0.2513, 4 split 0.2564): the layer-0 -> epilogue
// -> output-MMA chain and the narrow MMAs bound these kernels, not digitiser issue slots.
#ifndef LAKE_OTC_DIG_WARPS
#define LAKE_OTC_DIG_WARPS 2
#endif
#ifndef LAKE_OTC_DIG_TOP
#define LAKE_OTC_DIG_TOP 0
#endif
constexpr uint32_t kOtcDigWarps = LAKE_OTC_DIG_WARPS;
static_assert(kOtcDigWarps == 2 || kOtcDigWarps == 4, "128 rows over 64 or 128 digitiser threads");
constexpr bool kOtcDigTop = LAKE_OTC_DIG_TOP != 0;
template <bool OTC> constexpr uint32_t dig_warps() { return OTC ? kOtcDigWarps : 2u; }
template <bool OTC> constexpr uint32_t extra_warps() {
  return OTC ? (kOtcDigTop ? kOtcDigWarps : kOtcDigWarps - 2u) : 0u;
}
template <bool OTC> constexpr int threads_of() { return kThreads + 32 * (int)extra_warps<OTC>(); }

__device__ __forceinline__ uint32_t img_wh(int l, int prec) { return tc_wh_off(l, prec); }

// Column of TMEM (relative to the H buffer) where K-step s of the next layer's A operand
// sits. fp16/bf16: the warp's kEpiCols fp32 columns [col0, col0 + kEpiCols) are packed in
// place into kEpiCols/2 columns [col0, col0 + kEpiCols/2), so K-step s (features 16s..16s+15)
// is at packed column tmem_a_col(s). tf32: one value per column, in place: column 8s.
template <int PREC>
__host__ __device__ constexpr uint32_t tmem_a_col(uint32_t s) {
  if constexpr (PREC == 2) return s * 8;
  else return (s / (kEpiCols / 16)) * kEpiCols + (s % (kEpiCols / 16)) * 8;
}

// H chunk epilogue for one warp (H kept in TMEM): W fp32 accumulator columns of its 32 rows
// -> + bias (fp32, one rounding) -> ReLU + one rounding to the operand type -> written back
// in place into the accumulator it came from (see tmem_a_col), where the next layer's MMA
// reads it as its A operand (no SMEM H tile, no proxy fence).
// Layer 0's staged bias is zero: the MMA already added b0 (slot 31 of X is 1, W0's slot-31
// column is b0: DESIGN.md §2). One code path for every layer keeps the kernel's I-cache
// footprint down (a second, bias-free variant of the unrolled loops cost 10% at C5).
// fp16/bf16: every bias was added by the MMA (layer 0: W0's slot 31; hidden layers: the
// bias-block MMA), so the epilogue is ReLU + one rounding. tf32 adds the fp32 bias here.
template <int PREC, int W>
__device__ __forceinline__ void epi_to_h_tmem(const uint32_t (&r)[W], const float *bias,
                                              uint32_t col0, uint32_t tlane_base) {
  constexpr int NW = PREC == 2 ? W : W / 2;  // 32-bit words written back
  uint32_t p[NW];
#pragma unroll
  for (int c4 = 0; c4 < W / 4; ++c4) {
    float bb[4] = {0.0f, 0.0f, 0.0f, 0.0f};
    if constexpr (PREC == 2) {
      const float4 b4 = *reinterpret_cast<const float4 *>(bias + col0 + c4 * 4);
      bb[0] = b4.x; bb[1] = b4.y; bb[2] = b4.z; bb[3] = b4.w;
    }
#pragma unroll
    for (int e = 0; e < 4; e += 2) {
      const int c = c4 * 4 + e;
#ifdef LAKE_ABL_NOCVT  // timing-only ablation: no conversion arithmetic
      if constexpr (PREC == 2) { p[c] = r[c]; p[c + 1] = r[c + 1]; }
      else p[c / 2] = r[c] ^ r[c + 1];
#else
      const float v0 = PREC == 2 ? __uint_as_float(r[c]) + bb[e] : __uint_as_float(r[c]);
      const float v1 = PREC == 2 ? __uint_as_float(r[c + 1]) + bb[e + 1] : __uint_as_float(r[c + 1]);
      if constexpr (PREC == 2) {
        p[c] = ptx::relu_tf32(v0);
        p[c + 1] = ptx::relu_tf32(v1);
      } else if constexpr (PREC == 0) {
        p[c / 2] = ptx::relu_pack_f16(v0, v1);
      } else {
        p[c / 2] = ptx::relu_pack_bf16(v0, v1);
      }
#endif
    }
  }
#ifdef LAKE_ABL_NOST  // timing-only ablation: H not written back (never true at run time)
  if (p[0] == 0x12345678u && p[1] == 0x9abcdef0u)
#endif
  {
    if constexpr (NW == 32) ptx::tmem_st_32x32b_x32(tlane_base + col0, p);
    else if constexpr (NW == 16) ptx::tmem_st_32x32b_x16(tlane_base + col0, p);
    else if constexpr (NW == 8) ptx::tmem_st_32x32b_x8(tlane_base + col0, p);
    else ptx::tmem_st_32x32b_x4(tlane_base + col0, p);
  }
}

// ---- layer-0 A rows in the tensor-core slot order (tc_slot_digit, lake_internal.h) ----------
// Operand pair (a, b), small integers: the 16-bit pattern M | v is the value M' + v (fp16:
// 0x6400 = 1024, ulp 1 on [1024, 2048); bf16: 0x4300 = 128, ulp 1 on [128, 256)), so one
// packed subtract of (M', M') gives (a, b) exactly for a, b < 128.
template <int PREC>
__device__ __forceinline__ uint32_t pair_of(uint32_t a, uint32_t b) {
  constexpr uint32_t kMagic2 = PREC == 0 ? 0x64006400u : 0x43004300u;
  const uint32_t u = a | (b << 16) | kMagic2;
  return PREC == 0 ? ptx::sub_f16x2(u, kMagic2) : ptx::sub_bf16x2(u, kMagic2);
}
// tf32 (fp32 bits): 0x4B000000 | v is 2^23 + v exactly (v < 2^23), minus 2^23 gives v.
__device__ __forceinline__ uint32_t tf32_of(uint32_t v) {
  return __float_as_uint(__uint_as_float(0x4B000000u | v) - 8388608.0f);
}
template <int PREC>
struct XRow {
  uint32_t w[PREC == 2 ? 32 : 16];  // the row's 32 slots: pairs (fp16/bf16) or values (tf32)
};

// Raw record -> slot row by table lookups: each 4-digit field is hi = v / 100, lo = v % 100
// and two entries of the 100-pair table; each 3-digit field contributes its tail pair (lo)
// and its head digit (hi), heads paired at slots 26-30. D_w(v) = digits of min(v, 10^w - 1).
template <int PREC>
__device__ __forceinline__ void row_from_raw(const uint32_t (&rec)[9], const uint32_t *t100,
                                             XRow<PREC> &x) {
  uint32_t head[5];
#pragma unroll
  for (int f = 0; f < 4; ++f) {  // lat_us[f] -> slots 4f..4f+3
    const uint32_t v = rec[1 + f] < 9999u ? rec[1 + f] : 9999u;
    const uint32_t hi = v / 100u, lo = v - 100u * hi;
    if constexpr (PREC == 2) {
      x.w[4 * f + 0] = t100[2 * hi]; x.w[4 * f + 1] = t100[2 * hi + 1];
      x.w[4 * f + 2] = t100[2 * lo]; x.w[4 * f + 3] = t100[2 * lo + 1];
    } else {
      x.w[2 * f] = t100[hi];
      x.w[2 * f + 1] = t100[lo];
    }
  }
#pragma unroll
  for (int g = 0; g < 5; ++g) {  // q_now, q_hist[0..3] -> tail slots 16+2g, 17+2g; head 26+g
    const uint32_t r = g == 0 ? rec[0] : rec[4 + g];
    const uint32_t v = r < 999u ? r : 999u;
    const uint32_t hi = v / 100u, lo = v - 100u * hi;
    if constexpr (PREC == 2) {
      x.w[16 + 2 * g] = t100[2 * lo];
      x.w[17 + 2 * g] = t100[2 * lo + 1];
      x.w[26 + g] = tf32_of(hi);
    } else {
      x.w[8 + g] = t100[lo];
    }
    head[g] = hi;
  }
  if constexpr (PREC == 2) {
    x.w[31] = tf32_of(1);  // slot 31: the constant 1 that multiplies b0
  } else {
    x.w[13] = pair_of<PREC>(head[0], head[1]);
    x.w[14] = pair_of<PREC>(head[2], head[3]);
    x.w[15] = pair_of<PREC>(head[4], 1);  // slot 31: the constant 1 that multiplies b0
  }
}
// Packed row (slot-order nibbles, digitize.cuh) -> slot row: byte p is the pair of slots 2p,
// 2p+1.
template <int PREC>
__device__ __forceinline__ void row_from_packed(const uint4 v, XRow<PREC> &x) {
  const uint32_t q[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
  for (int p = 0; p < 16; ++p) {
    const uint32_t b = (q[p >> 2] >> (8 * (p & 3))) & 0xFFu;
    if constexpr (PREC == 2) {
      x.w[2 * p] = tf32_of(b & 0xFu);
      x.w[2 * p + 1] = tf32_of(b >> 4);
    } else {
      x.w[p] = pair_of<PREC>(b & 0xFu, b >> 4);
    }
  }
}
// Canonical-order values (LAKE_IN_DIGITS bytes; dg[31] = 1, the bias input) -> slot row. Digit bytes can be
// up to 255: exact in fp16 (< 1024) and tf32; bf16 pairs by conversion instead of the trick.
template <int PREC>
__device__ __forceinline__ void row_from_canonical(const uint32_t (&dg)[32], XRow<PREC> &x) {
#pragma unroll
  for (int s = 0; s < 32; s += 2) {
    const uint32_t a = dg[tc_slot_digit(s)], b = dg[tc_slot_digit(s + 1)];
    if constexpr (PREC == 2) {
      x.w[s] = tf32_of(a);
      x.w[s + 1] = tf32_of(b);
    } else if constexpr (PREC == 0) {
      x.w[s / 2] = pair_of<0>(a, b);
    } else {
      x.w[s / 2] = (uint32_t)__bfloat16_as_ushort(__uint2bfloat16_rn(a)) |
                   ((uint32_t)__bfloat16_as_ushort(__uint2bfloat16_rn(b)) << 16);
    }
  }
}

// Last hidden layer: ReLU(acc + b) in fp32, accumulated straight into the two logits
// (two partial sums per logit to halve the dependent-FMA chain). fp16/bf16: b is already
// in acc (bias MMA).
#ifdef LAKE_LOGITS_FFMA2
// A/B: paired form (fma.rn.f32x2): p[0]/p[2] and p[1]/p[3] are the two lanes of one 64-bit
// accumulator each, so every lane does exactly the scalar form's FMAs (same bits) in half the
// FMA issue slots. Measured slower at C5 (3.287 vs 3.264 ms): the packing moves cost more.
template <int PREC, int W>
__device__ __forceinline__ void epi_to_logits(const uint32_t (&r)[W], const float *bl,
                                              const float *wo, uint32_t col0, float (&p)[4]) {
  uint64_t a0 = ptx::pack_f32x2(p[0], p[2]), a1 = ptx::pack_f32x2(p[1], p[3]);
#pragma unroll
  for (int c4 = 0; c4 < W / 4; ++c4) {
    float bb[4] = {0.0f, 0.0f, 0.0f, 0.0f};
    if constexpr (PREC == 2) {
      const float4 b4 = *reinterpret_cast<const float4 *>(bl + col0 + c4 * 4);
      bb[0] = b4.x; bb[1] = b4.y; bb[2] = b4.z; bb[3] = b4.w;
    }
    const ulonglong2 w0 = *reinterpret_cast<const ulonglong2 *>(wo + col0 + c4 * 4);
    const ulonglong2 w1 = *reinterpret_cast<const ulonglong2 *>(wo + kHidden + col0 + c4 * 4);
    float h[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const float v = PREC == 2 ? __uint_as_float(r[c4 * 4 + e]) + bb[e] : __uint_as_float(r[c4 * 4 + e]);
      h[e] = v > 0.0f ? v : 0.0f;
    }
    const uint64_t h01 = ptx::pack_f32x2(h[0], h[1]), h23 = ptx::pack_f32x2(h[2], h[3]);
    ptx::fma_f32x2(a0, h01, w0.x);
    ptx::fma_f32x2(a1, h01, w1.x);
    ptx::fma_f32x2(a0, h23, w0.y);
    ptx::fma_f32x2(a1, h23, w1.y);
  }
  ptx::unpack_f32x2(a0, p[0], p[2]);
  ptx::unpack_f32x2(a1, p[1], p[3]);
}
#else
template <int PREC, int W>
__device__ __forceinline__ void epi_to_logits(const uint32_t (&r)[W], const float *bl,
                                              const float *wo, uint32_t col0, float (&p)[4]) {
#pragma unroll
  for (int c4 = 0; c4 < W / 4; ++c4) {
    float bb[4] = {0.0f, 0.0f, 0.0f, 0.0f};
    if constexpr (PREC == 2) {
      const float4 b4 = *reinterpret_cast<const float4 *>(bl + col0 + c4 * 4);
      bb[0] = b4.x; bb[1] = b4.y; bb[2] = b4.z; bb[3] = b4.w;
    }
    const float4 w0 = *reinterpret_cast<const float4 *>(wo + col0 + c4 * 4);
    const float4 w1 = *reinterpret_cast<const float4 *>(wo + kHidden + col0 + c4 * 4);
    const float ww0[4] = {w0.x, w0.y, w0.z, w0.w};
    const float ww1[4] = {w1.x, w1.y, w1.z, w1.w};
#pragma unroll
    for (int e = 0; e < 4; ++e) {
#ifdef LAKE_ABL_NOLOGITS  // timing-only ablation: no output-layer arithmetic
      p[e] += __uint_as_float(r[c4 * 4 + e]) + bb[e] + ww0[e] + ww1[e];
#else
      float h = PREC == 2 ? __uint_as_float(r[c4 * 4 + e]) + bb[e] : __uint_as_float(r[c4 * 4 + e]);
      h = h > 0.0f ? h : 0.0f;
      p[(e & 1) * 2 + 0] = fmaf(h, ww0[e], p[(e & 1) * 2 + 0]);
      p[(e & 1) * 2 + 1] = fmaf(h, ww1[e], p[(e & 1) * 2 + 1]);
#endif
    }
  }
}
#endif

template <int PREC, int IN_KIND, bool OTC>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(threads_of<OTC>(), 1)
mlp_tc_kernel(const void *__restrict__ in, const __grid_constant__ TileSched ts, int nh_layout,
              uint8_t *__restrict__ decisions, float *__restrict__ logits) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const Layout L = tc_layout(nh_layout, PREC);
  constexpr uint32_t kXB = x_bytes(PREC);
  constexpr uint32_t kKS = ksteps_per_chunk(PREC);  // MMA K-steps per H chunk
  constexpr uint32_t kK0S = kTcK0 / kmma(PREC);       // MMA K-steps of layer 0
  const uint32_t sbase = ptx::smem_u32(smem);
  const uint32_t bar0 = sbase + L.bar;
  auto bar = [&](uint32_t slot) { return bar0 + slot * 8; };
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ptx::cluster_ctarank();
  const uint32_t cid = ptx::cluster_id_x(), ncl = ptx::num_clusters_x();

#ifdef LAKE_TRACE
  unsigned long long *const tr_buf = g_lake_trace;  // read once: events cost no global load
#ifdef LAKE_TRACE_QUAD  // streams: epilogue warps 4, 5, 6, 3 of rank 0 (TMEM quadrants 0-3)
  int tr_stream = !(tr_buf && cid == 0 && rank == 0) || lane != 0 ? -1
                      : (warp >= kWarpEpi && warp < kWarpEpi + 4) ? (int)((warp - kWarpEpi + 3) & 3) : -1;
#elif defined(LAKE_TRACE_PAIR)  // streams: MMA, epilogue warp 3 of rank 0 / rank 1, warp 7 of rank 0
  int tr_stream = !(tr_buf && cid == 0) || lane != 0 ? -1
                      : (warp == kWarpMma && rank == 0) ? 0
                      : (warp == kWarpEpi && rank == 0) ? 1
                      : (warp == kWarpEpi && rank == 1) ? 2
                      : (warp == kWarpEpi + 4 && rank == 0) ? 3 : -1;
#elif defined(LAKE_TRACE_OTC)  // streams: MMA, the two epilogue groups' poller warps (rank 0), digitiser
  int tr_stream = !(tr_buf && cid == 0 && rank == 0) || lane != 0 ? -1
                      : warp == kWarpMma ? 0 : warp == kWarpEpi + 1 ? 1
                      : warp == kWarpEpi + kGroupWarps + 1 ? 2
                      : threadIdx.x == ((OTC && kOtcDigTop) ? (uint32_t)kThreads : 0u) ? 3 : -1;
#elif defined(LAKE_TRACE_DIG)  // streams: MMA, digitiser thread 0 of rank 0 / rank 1, epi warp 3
  int tr_stream = !(tr_buf && cid == 0) ? -1
                      : (warp == kWarpMma && lane == 0 && rank == 0) ? 0
                      : (threadIdx.x == 0 && rank == 0) ? 1
                      : (threadIdx.x == 0 && rank == 1) ? 2
                      : (warp == kWarpEpi && lane == 0 && rank == 0) ? 3 : -1;
#else
  int tr_stream = !(tr_buf && cid == 0 && rank == 0) ? -1
                      : (warp == kWarpMma && lane == 0) ? 0 : (warp == kWarpEpi && lane == 0) ? 1
                      : (warp == kWarpMma - 1 && lane == 0) ? 2 : (threadIdx.x == 0) ? 3 : -1;
#endif
  uint32_t tr_i = 0;
#ifdef LAKE_TRACE_SMEM
  const uint32_t tr_smem = sbase + L.total;
  if (tr_buf && cid == 0)  // clear the log (keys 0 = unused)
    for (uint32_t i = threadIdx.x; i < 4 * LAKE_TRACE_CAP * 4; i += blockDim.x)
      reinterpret_cast<uint32_t *>(smem + L.total)[i] = 0;
  if (PREC == 2) tr_stream = -1;
#endif
#endif
  const int64_t n_tiles = ts.n_tiles_dev ? (int64_t)*ts.n_tiles_dev : ts.n_tiles;
  int64_t t_lo = 0, t_hi = n_tiles;  // part 1 / 2: the NN-class prefix / the rest (multi)
  if (ts.part) {
    const int64_t sp = *ts.tile_split_dev < n_tiles ? (int64_t)*ts.tile_split_dev : n_tiles;
    if (ts.part == 1) t_hi = sp;
    else t_lo = sp;
  }
  const int64_t t_begin = t_lo + (t_hi - t_lo) * cid / ncl;
  const int64_t t_end = t_lo + (t_hi - t_lo) * (cid + 1) / ncl;

  if (threadIdx.x == 0) {
    ptx::mbar_init(bar(B_WLOAD), 1);
    ptx::mbar_init(bar(B_WREADY), 2);            // one arrive per CTA loader
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(bar(B_XFULL + i), 2);       // one arrive per CTA digitiser group
      ptx::mbar_init(bar(B_XEMPTY + i), 1);      // tcgen05.commit (multicast)
      ptx::mbar_init(bar(B_DFULL + i), 1);       // tcgen05.commit (multicast): H layers
      ptx::mbar_init(bar(B_DFULLX + i), 1);      // tcgen05.commit (multicast): last layer
      ptx::mbar_init(bar(B_DHALF + i), 1);       // tcgen05.commit (multicast): its first half
#ifdef LAKE_TEMPTY_AGG
      ptx::mbar_init(bar(B_TEMPTY + i), kGroupWarps + 1);  // leader's group warps + the peer
#else
      ptx::mbar_init(bar(B_TEMPTY + i), 2 * kGroupWarps);  // the draining group, both CTAs
#endif
    }
    for (uint32_t i = 0; i < kChunks; ++i) ptx::mbar_init(bar(B_HREADY + i), kHreadyCount);
    ptx::mbar_init(bar(B_WFREE), 1);             // tcgen05.commit (multicast)
    for (uint32_t i = 0; i < kTcRingSlots; ++i) {
      // leader: its own loader's arrive.expect_tx (+ bytes) and the peer's forwarded arrive;
      // peer: its loader's arrive.expect_tx (+ bytes)
      ptx::mbar_init(bar(B_RFULL + i), rank == 0 ? 2 : 1);
      ptx::mbar_init(bar(B_REMPTY + i), 1);      // tcgen05.commit (multicast)
    }
    for (int i = 0; i < 2; ++i) ptx::mbar_init(bar(B_SFULL + i), 1);  // expect_tx arrive
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(bar(B_HDONE + i), 2 * kGroupWarps);  // the draining group, both CTAs
      ptx::mbar_init(bar(B_DOUT + i), 1);                 // tcgen05.commit (multicast)
    }
    ptx::fence_mbar_init();
  }
  if (warp == kWarpLoad) {
    ptx::tmem_alloc_cg2(sbase + L.bar + kTmemSlot, 512);
    ptx::tmem_relinquish_cg2();
  }
  // the bias MMA's A operand (fp16/bf16): 128 rows x K 16, K column 0 = 1, zeros elsewhere
  if constexpr (PREC != 2) {
    uint32_t *ones = reinterpret_cast<uint32_t *>(smem + L.ones);
    constexpr uint32_t kOne = PREC == 0 ? 0x3C00u : 0x3F80u;
    for (uint32_t i = threadIdx.x; i < tc_bias_block_bytes(PREC) / 4; i += blockDim.x)
      // core layout: element (r, k) at (k/8)*2048 + r*16 + (k%8)*2; k = 0 <=> word r*4
      ones[i] = (i < 128 * 4 && (i & 3) == 0) ? kOne : 0u;
    ptx::fence_proxy_async_smem();  // generic-proxy writes read by the tensor core
  }
  // the digitisers' pair table: entry x = (x / 10, x % 10) in the operand type
  for (uint32_t x = threadIdx.x; x < 100; x += blockDim.x) {
    uint32_t *t100 = reinterpret_cast<uint32_t *>(smem + L.t100);
    if constexpr (PREC == 2) {
      t100[2 * x] = tf32_of(x / 10);
      t100[2 * x + 1] = tf32_of(x % 10);
    } else {
      t100[x] = pair_of<PREC>(x / 10, x % 10);
    }
  }
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + L.bar + kTmemSlot);

  if (warp == kWarpLoad) {
    // ================= weight loader (both CTAs) =================
    // Resident part of the model's image at model switches; for tf32 NN+2 also the W2
    // K-slices of every tile into the ring (kTcRingSlots x 8 KB, 16 slices per tile).
    if (lane == 0) {
      const uint8_t *cur = nullptr;
      uint32_t wl_phase = 0, wf_phase = 0;
      uint32_t rc = 0;  // ring slices issued
      const uint32_t wready_leader = ptx::mapa(bar(B_WREADY), 0);
      for (int64_t t = t_begin; t < t_end; ++t) {
        const TileInfo ti = tile_info<PREC>(ts, t);
        const uint8_t *src = ti.img + (size_t)rank * tc_image_bytes(ti.nh, PREC);
        if (ti.img != cur) {
          // Model switch: every MMA reading the old weights must have completed. The MMA
          // thread commits B_WFREE once per switch, after the old model's last MMA; it
          // cannot commit the next one before this loader has signalled B_WREADY.
          if (cur) {
            ptx::mbar_wait(bar(B_WFREE), wf_phase);
            wf_phase ^= 1;
          }
          const uint32_t bytes = tc_resident_bytes(ti.nh, PREC);
          ptx::mbar_arrive_expect_tx(bar(B_WLOAD), bytes);
          for (uint32_t off = 0; off < bytes; off += 32768) {
            const uint32_t len = (bytes - off) < 32768 ? (bytes - off) : 32768;
            ptx::bulk_g2s(sbase + off, src + off, len, bar(B_WLOAD));
          }
          ptx::mbar_wait(bar(B_WLOAD), wl_phase);
          wl_phase ^= 1;
          ptx::mbar_arrive_cluster(wready_leader);
          cur = ti.img;
        }
        if constexpr (PREC == 2) {
          if (streams_w2(ti.nh, PREC)) {
            const uint8_t *w2 = src + img_wh(2, PREC);
            for (uint32_t c = 0; c < tc_wh_half_bytes(PREC) / kTcRingSlotBytes; ++c, ++rc) {
              const uint32_t slot = rc % kTcRingSlots;
              if (rc >= kTcRingSlots)
                ptx::mbar_wait(bar(B_REMPTY + slot), ((rc / kTcRingSlots) - 1) & 1);
              ptx::mbar_arrive_expect_tx(bar(B_RFULL + slot), kTcRingSlotBytes);
              ptx::bulk_g2s(sbase + L.ring + slot * kTcRingSlotBytes, w2 + c * kTcRingSlotBytes,
                            kTcRingSlotBytes, bar(B_RFULL + slot));
            }
          }
        }
      }
    }
  } else if (warp == kWarpMma) {
    if constexpr (PREC == 2) {
      // ================= ring forwarder (peer CTA, one thread) =================
      // The leader's MMA reads both CTAs' W2 halves, but may only wait on its own
      // mbarriers: forward each completed peer slice to the leader's B_RFULL.
      if (rank == 1 && lane == 0) {
        const uint32_t rfull_leader0 = ptx::mapa(bar(B_RFULL), 0);
        uint32_t fc = 0;
        for (int64_t t = t_begin; t < t_end; ++t) {
          const TileInfo ti = tile_info<PREC>(ts, t);
          if (!streams_w2(ti.nh, PREC)) continue;
          for (uint32_t c = 0; c < tc_wh_half_bytes(PREC) / kTcRingSlotBytes; ++c, ++fc) {
            const uint32_t slot = fc % kTcRingSlots;
            ptx::mbar_wait(bar(B_RFULL + slot), (fc / kTcRingSlots) & 1);
            ptx::mbar_arrive_cluster(rfull_leader0 + slot * 8);
          }
        }
      }
    }
    // ================= MMA issuer (leader CTA) =================
    // The whole warp runs the schedule in converged, warp-uniform code (operands in uniform
    // registers); only the tcgen05.mma / commit issue is predicated on lane 0. A lane-0-only
    // region made the compiler wrap every MMA in an R2UR.BROADCAST waterfall loop whose
    // latency, not the tensor pipe, set the issue rate (ncu: fixed-latency stalls there).
    if (rank == 0) {
      const bool issuer = lane == 0;
      const uint32_t tm = __shfl_sync(0xffffffffu, tmem, 0);  // provably warp-uniform
#ifdef LAKE_ABL_HALFN  // timing-only ablation: hidden-layer MMAs with N = 128 (half the work)
      const uint32_t idesc = ptx::umma_idesc_f16(PREC, 256, 128);
#else
      const uint32_t idesc = ptx::umma_idesc_f16(PREC, 256, 256);
#endif
      // descriptors: one MMA K-step (16 fp16/bf16 or 8 tf32 = 32 B) = +2 core matrices =
      // +2*LBO bytes, i.e. +(2*LBO)>>4 in the 14-bit start-address field (no carry: SMEM <
      // 256 KB)
      constexpr uint64_t kStep = (2 * kLboR128) >> 4;
      const uint64_t xdesc0 = ptx::umma_desc(sbase + L.x, kLboR128, 128);
      const uint64_t xdesc1 = ptx::umma_desc(sbase + L.x + kXB, kLboR128, 128);
      const uint64_t w0desc = ptx::umma_desc(sbase, kLboR128, 128);
      const uint64_t ringdesc = ptx::umma_desc(sbase + L.ring, kLboR128, 128);
      const uint64_t onesdesc = ptx::umma_desc(sbase + L.ones, kLboR128, 128);
      uint64_t whdesc[kMaxHiddenLayers];
      for (int l = 1; l < kMaxHiddenLayers; ++l)
        whdesc[l] = ptx::umma_desc(sbase + img_wh(l, PREC), kLboR128, 128);
      const uint8_t *cur = nullptr;
      uint32_t w_phase = 0, g = 0, h_phase = 0, t_phase = 0;  // h/t_phase: one bit per slot
      uint32_t used = 0;  // bit b: accumulator b has been written before
      uint32_t mc = 0;    // ring slices consumed
      int64_t it = 0;
      auto acquire_buf = [&](uint32_t b) {  // accumulator b must be drained by the epilogues
        if (used & (1u << b)) {
          ptx::mbar_wait(bar(B_TEMPTY + b), (t_phase >> b) & 1);
          t_phase ^= (1u << b);
        }
        used |= (1u << b);
      };
      TileInfo nxt;
      if (t_begin < t_end) nxt = tile_info<PREC>(ts, t_begin);
      // schedule entries two tiles ahead: the model slot of tile t+2 is loaded at the top of
      // tile t and the dependent model-table loads of tile t+1 are issued there too, from a
      // slot loaded one tile earlier, so no load result is waited for on the tile boundary
      auto slot_of = [&](int64_t tt) -> int32_t { return ts.tile_model ? ts.tile_model[tt] : -1; };
      int32_t slot_n = (t_begin + 1 < t_end) ? slot_of(t_begin + 1) : -1;
      for (int64_t t = t_begin; t < t_end; ++t, ++it) {
        LAKE_TEV(T_TOP, it, 0, 0);
        const TileInfo ti = nxt;
        const int32_t slot_nn = (t + 2 < t_end) ? slot_of(t + 2) : -1;
        if (t + 1 < t_end) {
          const DevModel *mm = slot_n >= 0 ? &ts.table[slot_n] : &ts.model;
          nxt.model = mm;
          nxt.img = mm->tc_img[PREC];
          nxt.nh = mm->nh < ts.nh_cap ? mm->nh : ts.nh_cap;
        }
        slot_n = slot_nn;
        LAKE_TEV(T_SCHED, it, 0, 0);
        if (ti.img != cur) {
          ptx::mbar_wait(bar(B_WREADY), w_phase);
          w_phase ^= 1;
          cur = ti.img;
        }
        LAKE_TEV(T_WREADY, it, 0, 0);
        const int nh = OTC ? 1 : ti.nh;  // an out_on_tc kernel only runs NN tiles
        const bool stream = streams_w2(nh, PREC);
        const uint32_t xb = (uint32_t)(it & 1);
        {  // layer 0: D = X[128(x2) x 32] * W0^T
          const uint32_t b = g & 1;
          acquire_buf(b);
          LAKE_TEV(T_TEMPTY, it, 0, 0);
          ptx::mbar_wait(bar(B_XFULL + xb), (uint32_t)((it >> 1) & 1));
          LAKE_TEV(T_XFULL, it, 0, 0);
          ptx::tc_fence_after();
          const uint32_t d = tm + b * 256;
          const uint64_t xd = xb ? xdesc1 : xdesc0;
#pragma unroll
          for (uint32_t s = 0; s < kK0S; ++s) {
            if (issuer) ptx::mma_cg2<PREC>(d, xd + s * kStep, w0desc + s * kStep, idesc, s);
            LAKE_TEV(T_MMA0, it, 0, s);
          }
          if (issuer) ptx::mma_commit_cg2(bar(B_XEMPTY + xb), 0x3);
          LAKE_TEV(T_CX, it, 0, 0);
          // NN: the accumulator's buffer picks the draining group (b0 -> group 0, b1 -> 1),
          // so both groups convert logits and two NN tiles are drained at once
          if (issuer)
            ptx::mma_commit_cg2(bar((kEpiGroups == 2 && nh == 1 && b == 1 ? B_DFULLX : B_DFULL) + b),
                                0x3);
          __syncwarp();
          LAKE_TEV(T_COMMIT, it, 0, 0);
          ++g;
        }
        for (int l = 1; l < nh; ++l) {  // hidden layers 1..nh-1 (K = 256)
          const uint32_t b = g & 1;
          acquire_buf(b);
          LAKE_TEV(T_TEMPTY, it, l, 0);
          ptx::tc_fence_after();
          const uint32_t d = tm + b * 256;
          // A = H(l-1), in place in the previous layer's accumulator buffer
          const uint32_t ha = tm + ((g - 1) & 1) * 256;
          const bool from_ring = stream && l == 2;
          const uint64_t wd = l == 1 ? whdesc[1] : whdesc[2];
          // fp16/bf16: the layer's bias first (D = ones x bias-block^T initialises the
          // accumulator; it needs no H, so it is issued before the first chunk wait)
          constexpr uint32_t kAcc = PREC == 2 ? 0u : 1u;
          const bool split = kL2Split && PREC != 2 && l + 1 == nh;
          // N = 128 halves: B rows 64..127 of each CTA's image start 8 row groups (1 KB) in
          constexpr uint32_t kHalfB = (8u * 128u) >> 4;
          const uint32_t idesc_h = ptx::umma_idesc_f16(PREC, 256, 128);
          if constexpr (PREC != 2)
            if (issuer)
              ptx::mma_cg2<PREC>(d, onesdesc, wd + (tc_wh_half_bytes(PREC) >> 4),
                                 split ? idesc_h : idesc, 0);
          for (uint32_t kc = 0; kc < kChunks; ++kc) {
#ifndef LAKE_ABL_NOHREADY  // timing-only ablation: the MMA never waits for H chunks
            ptx::mbar_wait(bar(B_HREADY + kc), (h_phase >> kc) & 1);
#endif
            h_phase ^= (1u << kc);
            LAKE_TEV(T_HREADY, it, l, kc);
            ptx::tc_fence_after();
            if (from_ring) {
              // W2 K-slices from the ring: one 8-KB slot = 16 K = 2 tf32 K-steps
              constexpr uint32_t kSPS = kTcRingSlotBytes / (2 * kLboR128);  // K-steps per slot
#pragma unroll
              for (uint32_t s = 0; s < kKS; ++s) {
                const uint32_t ks = kc * kKS + s;
                const uint32_t slot = mc % kTcRingSlots;
                if (s % kSPS == 0) {
                  ptx::mbar_wait(bar(B_RFULL + slot), (mc / kTcRingSlots) & 1);
                  ptx::tc_fence_after();
                }
                if (issuer)
                  ptx::mma_cg2_ts<PREC>(d, ha + tmem_a_col<PREC>(ks),
                                      ringdesc + (slot * kTcRingSlotBytes >> 4) + (s % kSPS) * kStep,
                                      idesc, ks | kAcc);
                if (s % kSPS == kSPS - 1) {
                  if (issuer) ptx::mma_commit_cg2(bar(B_REMPTY + slot), 0x3);
                  ++mc;
                }
              }
            } else {
#pragma unroll
              for (uint32_t s = 0; s < kKS; ++s) {
                const uint32_t ks = kc * kKS + s;
                if (issuer)
                  ptx::mma_cg2_ts<PREC>(d, ha + tmem_a_col<PREC>(ks), wd + ks * kStep,
                                        split ? idesc_h : idesc, ks | kAcc);
              }
            }
            __syncwarp();
            LAKE_TEV(T_ISSUED, it, l, kc);
          }
          if (split) {
            // first half (columns 0..127) complete -> the logits group starts on it; the
            // second half reuses the H chunks already waited for
            if (issuer) {
              ptx::mma_commit_cg2(bar(B_DHALF + b), 0x3);
              ptx::mma_cg2<PREC>(d + 128, onesdesc, wd + (tc_wh_half_bytes(PREC) >> 4) + kHalfB,
                                 idesc_h, 0);
            }
#pragma unroll 1
            for (uint32_t ks = 0; ks < kKS * kChunks; ++ks)
              if (issuer)
                ptx::mma_cg2_ts<PREC>(d + 128, ha + tmem_a_col<PREC>(ks), wd + ks * kStep + kHalfB,
                                      idesc_h, 1u);
            __syncwarp();
          }
          if (issuer)
            ptx::mma_commit_cg2(bar((kEpiGroups == 2 && l + 1 == nh ? B_DFULLX : B_DFULL) + b), 0x3);
          __syncwarp();
          LAKE_TEV(T_COMMIT, it, l, 0);
          ++g;
        }
        const bool wswitch = t + 1 < t_end && nxt.img != cur;
        if (wswitch && issuer) ptx::mma_commit_cg2(bar(B_WFREE), 0x3);  // old weights no longer read
        __syncwarp();
      }
    }
  } else if (OTC ? (kOtcDigTop ? warp >= (uint32_t)kThreads / 32
                                : (warp >= kWarpDig && warp < kWarpDig + 2) || warp >= (uint32_t)kThreads / 32)
                 : (warp >= kWarpDig && warp < kWarpDig + 2)) {
    // ================= digitisers: input rows -> X (operand-type digits) ===============
    // Each CTA's 128 rows of a tile are contiguous in one of three staged formats, brought
    // into SMEM by a bulk copy (cp.async.bulk, TMA engine) two tiles ahead and converted from
    // there (2 rows per thread):
    //   packed  multi-model calls: the grouping pass wrote every I/O's packed digit row
    //           (16 B, digitize.cuh) in model-grouped order -> ts.pdig
    //   raw     single-model calls, LAKE_IN_RAW, 16-B aligned input: 36-B records
    //   digits  single-model calls, LAKE_IN_DIGITS, 16-B aligned input: 32-B rows
    // Anything else (misaligned input, or rows too large for this precision's staging
    // buffers) gathers each row with global loads (the fallback below).
    constexpr uint32_t ND = 32 * dig_warps<OTC>();  // digitiser threads
    constexpr uint32_t RPT = 128 / ND;                // rows per thread: d, d + ND
    const uint32_t d = (OTC && kOtcDigTop) ? threadIdx.x - (uint32_t)kThreads
                       : warp < (uint32_t)kThreads / 32 ? threadIdx.x - kWarpDig * 32
                                                        : 64u + threadIdx.x - (uint32_t)kThreads;
    const uint32_t xfull_leader0 = ptx::mapa(bar(B_XFULL), 0);
    const uint32_t row_bytes = ts.pdig ? 16u : (IN_KIND == LAKE_IN_RAW ? 36u : 32u);
#ifdef LAKE_ABL_NOSTAGE  // A/B switch: always the gather path
    const bool staged = false;
#else
    const bool staged = ts.pdig != nullptr ||
                        (ts.perm == nullptr && (reinterpret_cast<uintptr_t>(in) & 15) == 0 &&
                         128u * row_bytes <= kStageBytes(PREC));
#endif
    const uint8_t *stage_src = ts.pdig ? reinterpret_cast<const uint8_t *>(ts.pdig)
                                       : static_cast<const uint8_t *>(in);
    // rows of tile t in this CTA, and the 16-B-multiple prefix the bulk copy moves
    auto rows_of = [&](const TileInfo &ti) {
      const int r = ti.count - (int)(rank * 128);
      return (uint32_t)(r < 0 ? 0 : (r > 128 ? 128 : r));
    };
    auto issue = [&](int64_t t, uint32_t buf) {  // one thread
      const TileInfo ti = tile_info<PREC>(ts, t);
      const uint32_t bulk = (rows_of(ti) * row_bytes) & ~15u;
      if (bulk) {
        ptx::mbar_arrive_expect_tx(bar(B_SFULL + buf), bulk);
        ptx::bulk_g2s(sbase + L.stage + buf * kStageBytes(PREC),
                      stage_src + (size_t)(ti.begin + rank * 128) * row_bytes, bulk,
                      bar(B_SFULL + buf));
      } else {
        ptx::mbar_arrive(bar(B_SFULL + buf));
      }
    };
    if (staged && d == 0) {
      if (t_begin < t_end) issue(t_begin, 0);
      if (t_begin + 1 < t_end) issue(t_begin + 1, 1);
    }
    const uint32_t *t100 = reinterpret_cast<const uint32_t *>(smem + L.t100);
    int64_t it = 0;
    for (int64_t t = t_begin; t < t_end; ++t, ++it) {
      const TileInfo ti = tile_info<PREC>(ts, t);
      const uint32_t xb = (uint32_t)(it & 1);
      const uint32_t rows = rows_of(ti);
      XRow<PREC> xr[RPT];  // rows d (and d + 64) in the slot order
      if (staged) {
        const uint32_t sb = (uint32_t)(it & 1);
#ifndef LAKE_DIG_POLL_ALL
        if (d < 32) ptx::mbar_wait(bar(B_SFULL + sb), (uint32_t)((it >> 1) & 1));
        ptx::named_bar_sync(1, ND);
#else
        ptx::mbar_wait(bar(B_SFULL + sb), (uint32_t)((it >> 1) & 1));
#endif
        LAKE_TEV(T_XEMPTY, it, 1, 0);
        const uint32_t bulk = (rows * row_bytes) & ~15u;
        const uint8_t *st = smem + L.stage + sb * kStageBytes(PREC);
#pragma unroll
        for (int half = 0; half < (int)RPT; ++half) {
          const uint32_t r = d + ND * half;
          const bool valid = r < rows;
#ifdef LAKE_ABL_NODIG  // timing-only ablation: no digitiser conversion (staged inputs)
#pragma unroll
          for (int i = 0; i < (PREC == 2 ? 32 : 16); ++i) xr[half].w[i] = r + i + st[0];
          if (true) continue;
#endif
          if (ts.pdig) {
            row_from_packed<PREC>(valid ? *reinterpret_cast<const uint4 *>(st + r * 16)
                                        : make_uint4(0, 0, 0, 0), xr[half]);
          } else if (IN_KIND == LAKE_IN_RAW) {
            uint32_t rec[9];
            if (!valid) {
#pragma unroll
              for (int f = 0; f < 9; ++f) rec[f] = 0;
            } else if ((r + 1) * 36 <= bulk) {
              const uint32_t *src = reinterpret_cast<const uint32_t *>(st + r * 36);
#pragma unroll
              for (int f = 0; f < 9; ++f) rec[f] = src[f];
            } else {  // tail rows past the 16-B-multiple prefix: straight from global
              const uint32_t *src = reinterpret_cast<const uint32_t *>(in) +
                                    (size_t)(ti.begin + rank * 128 + r) * 9;
#pragma unroll
              for (int f = 0; f < 9; ++f) rec[f] = __ldg(src + f);
            }
            row_from_raw<PREC>(rec, t100, xr[half]);
          } else {
            uint32_t dg[32];
            uint4 v0 = make_uint4(0, 0, 0, 0), v1 = v0;
            if (valid) {
              v0 = *reinterpret_cast<const uint4 *>(st + r * 32);
              v1 = *reinterpret_cast<const uint4 *>(st + r * 32 + 16);
            }
            const uint32_t x[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
#pragma unroll
            for (int k = 0; k < 32; ++k) dg[k] = k < 31 ? (x[k >> 2] >> ((k & 3) * 8)) & 0xFFu : 1u;
            row_from_canonical<PREC>(dg, xr[half]);
          }
        }
#ifndef LAKE_DIG_POLL_ALL  // one polling warp (see the epilogue's accumulator-full wait)
        if (d < 32) ptx::mbar_wait(bar(B_XEMPTY + xb), (uint32_t)(((it >> 1) & 1) ^ 1));
        ptx::named_bar_sync(1, ND);
#else
        ptx::mbar_wait(bar(B_XEMPTY + xb), (uint32_t)(((it >> 1) & 1) ^ 1));
#endif
        LAKE_TEV(T_XEMPTY, it, 0, 0);
      } else {
        // gather fallback: both rows' loads are issued before any shared store (the
        // st.shared asm carries a memory clobber, so later loads could not be hoisted)
        uint32_t rec[RPT][9];
        // NN tiles (one tensor-core layer) are digitiser-bound: gather first, then wait.
        const bool early = ti.nh == 1;
        if (!early) ptx::mbar_wait(bar(B_XEMPTY + xb), (uint32_t)(((it >> 1) & 1) ^ 1));
#pragma unroll
        for (int half = 0; half < (int)RPT; ++half) {
          const uint32_t r = d + ND * half;
          const bool valid = r < rows;
          const int64_t p = ti.begin + rank * 128 + (valid ? r : 0);
          const int64_t io = ts.perm ? (int64_t)ts.perm[p] : p;
          if (IN_KIND == LAKE_IN_RAW) {
            const uint32_t *src = reinterpret_cast<const uint32_t *>(in) + io * 9;
#pragma unroll
            for (int f = 0; f < 9; ++f) rec[half][f] = valid ? __ldg(src + f) : 0u;
          } else {
            const uint4 *src = reinterpret_cast<const uint4 *>(
                reinterpret_cast<const uint8_t *>(in) + io * 32);
            uint4 v0 = make_uint4(0, 0, 0, 0), v1 = v0;
            if (valid) {
              v0 = __ldg(src);
              v1 = __ldg(src + 1);
            }
            rec[half][0] = v0.x; rec[half][1] = v0.y; rec[half][2] = v0.z; rec[half][3] = v0.w;
            rec[half][4] = v1.x; rec[half][5] = v1.y; rec[half][6] = v1.z; rec[half][7] = v1.w;
            rec[half][8] = 0;
          }
        }
        if (early) ptx::mbar_wait(bar(B_XEMPTY + xb), (uint32_t)(((it >> 1) & 1) ^ 1));
        LAKE_TEV(T_XEMPTY, it, 0, 0);
#pragma unroll
        for (int half = 0; half < (int)RPT; ++half) {
          if (IN_KIND == LAKE_IN_RAW) {
            row_from_raw<PREC>(rec[half], t100, xr[half]);
          } else {
            uint32_t dg[32];
#pragma unroll
            for (int k = 0; k < 32; ++k) dg[k] = k < 31 ? (rec[half][k >> 2] >> ((k & 3) * 8)) & 0xFFu : 1u;
            row_from_canonical<PREC>(dg, xr[half]);
          }
        }
      }
      // an absent row (ragged tile) stores zeros (raw: digits of all-zero fields are zero;
      // gathered invalid rows read 0s above)
      const uint32_t xs = sbase + L.x + xb * kXB;
#pragma unroll
      for (int half = 0; half < (int)RPT; ++half) {
        const uint32_t r = d + ND * half;
        constexpr int NKG = PREC == 2 ? 8 : 4;  // 16-B core-matrix groups per row
#pragma unroll
        for (int kg = 0; kg < NKG; ++kg)
          ptx::st_shared_v4(xs + kg * kLboR128 + r * 16, xr[half].w[kg * 4 + 0],
                            xr[half].w[kg * 4 + 1], xr[half].w[kg * 4 + 2], xr[half].w[kg * 4 + 3]);
      }
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(1, ND);  // X written; staging buffer it&1 fully read
      if (d == 0) {
        ptx::mbar_arrive_cluster(xfull_leader0 + xb * 8);
        if (staged && t + 2 < t_end) issue(t + 2, (uint32_t)(it & 1));
      }
      LAKE_TEV(T_XARRIVE, it, 0, 0);
    }
  } else if (warp >= kWarpEpi && warp < kWarpEpi + kEpiWarps) {
    // ================= epilogue =================
    constexpr uint32_t NG = kGroupWarps * 32;         // threads per epilogue group
    constexpr int W = kEpiCols;
    const uint32_t gy = (warp - kWarpEpi) / kGroupWarps;  // 0: H layers (or all), 1: last layer
    const uint32_t lw = (warp - kWarpEpi) % kGroupWarps;
    const uint32_t et = lw * 32 + lane;                   // thread index within the group
    const uint32_t q = warp & 3;                      // TMEM lane quadrant this warp may access
    const uint32_t hh = lw >> 2;                      // which W-column slice of each chunk
    const uint32_t row = q * 32 + lane;     // row within this CTA's 128
    const bool do_h = kEpiGroups == 1 || gy == 0;     // converts H-producing layers
    const bool do_last = kEpiGroups == 1 || gy == 1;  // converts the last layer
    const uint32_t hready_leader0 = ptx::mapa(bar(B_HREADY), 0);
    const uint32_t tempty_leader0 = ptx::mapa(bar(B_TEMPTY), 0);
    uint32_t do_phase = 0, hd_phase = 0;  // out_on_tc: B_DOUT / B_HDONE phases per buffer
    const uint32_t hdone_leader0 = ptx::mapa(bar(B_HDONE), 0);
    const DevModel *wcur = nullptr;  // out_on_tc: model of this group's W_out block
    const bool own0 = kEpiGroups == 2 && gy == 0;  // group 0's private output-layer copy
    float *prm = reinterpret_cast<float *>(smem + (own0 ? L.prm0 : L.prm));  // last b | W_out | b_out
    float *hbias = reinterpret_cast<float *>(smem + L.prm + kPrmFloats * 4);  // H-layer biases
    float *red = reinterpret_cast<float *>(smem + (own0 ? L.red0 : L.red));
    const uint32_t red_bar = (own0 ? 8 : 4) + q;  // named barrier of this quadrant's reduction
    // this warp has read accumulator b: arrive on its TEMPTY (leader CTA). LAKE_TEMPTY_AGG: the
    // peer CTA's group arrives once (named barrier 12 + group, then one remote arrive) and the
    // leader's warps through the CTA-local address
    auto release_acc = [&](uint32_t bb) {
#ifdef LAKE_TEMPTY_AGG
      if (rank == 0) {
        if (lane == 0) ptx::mbar_arrive(bar(B_TEMPTY + bb));
      } else {
        ptx::named_bar_sync(12 + gy, NG);
        if (et == 0) ptx::mbar_arrive_cluster(tempty_leader0 + bb * 8);
      }
#else
      if (lane == 0) ptx::mbar_arrive_cluster(tempty_leader0 + bb * 8);
#endif
    };
    const DevModel *cur = nullptr;
    uint32_t g = 0, d_phase = 0, dx_phase = 0;  // phase bits per accumulator buffer
    uint32_t dh_phase = 0;                      // LAKE_L2_NSPLIT: B_DHALF phases
    int64_t it = 0;
    TileInfo nxt;
    if (t_begin < t_end) nxt = tile_info<PREC>(ts, t_begin);
    for (int64_t t = t_begin; t < t_end; ++t, ++it) {
      const TileInfo ti = nxt;
      if (t + 1 < t_end) nxt = tile_info<PREC>(ts, t + 1);
      const int nh = OTC ? 1 : ti.nh;  // an out_on_tc kernel only runs NN tiles
      if (ti.model != cur) {
        // stage this model's epilogue parameters (each group the ones it uses): fp32 biases
        // of the H layers, fp32 last-layer bias | W_out | b_out
        ptx::named_bar_sync(2 + gy, NG);
        if (do_h) {
          for (uint32_t i = et; i < (uint32_t)(nh - 1) * kHidden / 4; i += NG)
            reinterpret_cast<float4 *>(hbias)[i] =
                i < kHidden / 4 ? make_float4(0.0f, 0.0f, 0.0f, 0.0f)  // b0: added by the MMA
                                : __ldg(reinterpret_cast<const float4 *>(ti.model->b[0]) + i);
        }
        if (do_last || (kEpiGroups == 2 && nh == 1)) {
          const float4 *src = reinterpret_cast<const float4 *>(ti.model->b[nh - 1]);
          // (split last layer: b_last and W_out rows staged in accumulator-column order)
          const bool perm_cols = kL2Split && PREC != 2 && nh >= 2;
          for (uint32_t i = et; i < kPrmFloats / 4; i += NG) {  // NN: b0 is added by the MMA
            uint32_t si = i;
            if (perm_cols && i < 3 * kHidden / 4)
              si = (i / (kHidden / 4)) * (kHidden / 4) + nsplit_feature(4 * (i % (kHidden / 4))) / 4;
            reinterpret_cast<float4 *>(prm)[i] = (nh == 1 && i < kHidden / 4)
                                                     ? make_float4(0.0f, 0.0f, 0.0f, 0.0f)
                                                     : __ldg(src + si);
          }
        }
        ptx::named_bar_sync(2 + gy, NG);
        cur = ti.model;
      }
      const float *wo = prm + kHidden;
      for (int l = 0; l < nh; ++l, ++g) {
        const bool last = (l + 1 == nh);
        const uint32_t b = g & 1;
        const bool nn2 = kEpiGroups == 2 && nh == 1;  // NN: buffer b is drained by group b
        if (nn2 ? gy != b : !(last ? do_last : do_h)) continue;
        {
          const bool x = kEpiGroups == 2 && (nn2 ? b == 1 : last);
          // split last layer: start on its first half (B_DHALF); B_DFULLX is waited mid-way
          const bool hx = kL2Split && PREC != 2 && last && nh >= 2;
          const uint32_t wb = hx ? bar(B_DHALF + b) : x ? bar(B_DFULLX + b) : bar(B_DFULL + b);
          const uint32_t wp = ((hx ? dh_phase : x ? dx_phase : d_phase) >> b) & 1;
#ifndef LAKE_EPI_POLL_ALL
          // One warp of the group polls the mbarrier (warp lw = 1: not on the MMA warp's SM
          // sub-partition), the others wait on the group's named barrier. Eight warps spinning
          // on try_wait took issue slots and SYNCS bandwidth from the MMA issuer: C5 fused
          // kernel 3.59 -> 3.34 ms with one poller (a __nanosleep backoff instead: 4.07 ms).
          if (lw == 1) ptx::mbar_wait(wb, wp);
          ptx::named_bar_sync(2 + gy, NG);
#else
          ptx::mbar_wait(wb, wp);
#endif
          if (hx) dh_phase ^= (1u << b);
          else if (x) dx_phase ^= (1u << b);
          else d_phase ^= (1u << b);
        }
        LAKE_TEV(T_DFULL, it, l, warp);
        ptx::tc_fence_after();
        const uint32_t tbase = tmem + ((q * 32) << 16) + b * 256;
        // j-th chunk's first column handled by this warp
        auto col_of = [&](uint32_t j) { return j * kChunkCols + hh * W; };
        const float *bl = prm;  // last-layer bias
        constexpr bool kPrefetch = W <= 32;  // two W-register buffers
        uint32_t ra[W], rb[W];  // rb unused (eliminated) without prefetch
// (layer 0's staged biases are zero: the MMA added b0; one code path keeps the unrolled
// chunk loop small - two variants cost ~40% more instructions and I-cache misses)
#define EPI_H(R) epi_to_h_tmem<PREC, W>(R, hbias + l * kHidden, col0, tbase)
// (NN: the staged last-layer bias is b0, zeroed at staging because the MMA added it)
#define EPI_L(R) epi_to_logits<PREC, W>(R, bl, wo, col0, p)
        ptx::tmem_ld_cols<W>(tbase + col_of(0), ra);
        ptx::tmem_ld_wait();
        if (!last) {
          // hidden layer feeding another MMA; with two register buffers the TMEM load of the
          // warp's next chunk is in flight while the current one is converted and stored
#pragma unroll kEpiUnroll
          for (uint32_t j = 0; j < kWarpChunks; ++j) {
            const uint32_t kc = j, col0 = col_of(j);
            if constexpr (kPrefetch) {
              if (j + 1 < kWarpChunks) {
                if (j & 1) ptx::tmem_ld_cols<W>(tbase + col_of(j + 1), ra);
                else ptx::tmem_ld_cols<W>(tbase + col_of(j + 1), rb);
              }
              if (j & 1) EPI_H(rb);
              else EPI_H(ra);
            } else {
              if (j > 0) {
                ptx::tmem_ld_cols<W>(tbase + col0, ra);
                ptx::tmem_ld_wait();
              }
              EPI_H(ra);
            }
            LAKE_TEV(T_STS, it, l, kc);
            ptx::tmem_st_wait();
            ptx::tc_fence_before();
            LAKE_TEV(T_FENCE, it, l, kc);
            __syncwarp();
#if defined(LAKE_HREADY_AGG)  // the peer CTA's group arrives once per chunk (see kHreadyCount)
            if (rank == 0) {
              if (lane == 0) ptx::mbar_arrive(bar(B_HREADY + kc));
            } else {
              ptx::named_bar_sync(12, NG);
              if (et == 0) ptx::mbar_arrive_cluster(hready_leader0 + kc * 8);
            }
#elif defined(LAKE_HREADY_LOCAL)  // A/B: the leader CTA's warps arrive through the CTA-local address
            if (lane == 0) {
              if (rank == 0) ptx::mbar_arrive(bar(B_HREADY + kc));
              else ptx::mbar_arrive_cluster(hready_leader0 + kc * 8);
            }
#else
            if (lane == 0) ptx::mbar_arrive_cluster(hready_leader0 + kc * 8);
#endif
            LAKE_TEV(T_CHUNK, it, l, kc);
            if (kPrefetch && j + 1 < kWarpChunks) ptx::tmem_ld_wait();
            LAKE_TEV(T_LDWAIT, it, l, kc);
          }
        } else if (OTC) {  // (every tile of an out_on_tc kernel is an NN tile)
          // NN, output layer on the tensor cores: H -> ReLU -> fp16/bf16, packed in place (the
          // A operand of the output MMA, as for a hidden layer); then this group's leader-CTA
          // poller issues the output layer once the whole group (both CTAs) has packed H. An
          // M=256 MMA costs >= 64 cycles whatever its N (scripts/microbench/umma_rate.cu), so
          // the 16 N=16 K-steps take ~1k tensor cycles; issued by the layer-0 thread they
          // blocked it that long, here they queue while layer 0 of later tiles goes on. Buffer
          // reuse stays ordered by TEMPTY: the group releases the accumulator only after
          // reading the result (DOUT). (Issuing the K-steps chunk by chunk as the packing
          // progresses measured 30% slower: per-chunk group barriers on the packing path.)
          const int pos = (int)(rank * 128 + row);
          const int64_t pp = ti.begin + pos;
          // the row's output index (multi-model calls): loaded now, first used after the
          // packing and the output MMA (opaque_u32 below) - its sign extension right after the
          // load put a DRAM latency in front of the packing (ncu: 14% of stall samples, C4)
          const uint32_t io_ld = (ts.perm && pos < ti.count) ? (uint32_t)__ldg(ts.perm + pp) : 0u;
          static_assert(!OTC || (kEpiCols == 16 && kChunks == 8 && kEpiPerQ == 2), "OTC packing layout");
          if (ti.model != wcur) {
            // this group's W_out block, rewritten whole (the region held another model's
            // weights in between): leader CTA rows 0, 1 = W_out, zeros elsewhere. Safe here:
            // the accumulator is full, so this model's weights are resident and every MMA of
            // an earlier model (and this group's previous output MMA) has completed.
            const float *wsrc = ti.model->b[0] + kHidden;  // NN: b0 | W_out[2][256] | b_out
            uint32_t *wblk = reinterpret_cast<uint32_t *>(smem + L.wout + gy * kWoutBytes);
            for (uint32_t i = et; i < kWoutBytes / 4; i += NG) {
              // word i: core column kc = i / 32, row r = (i / 4) % 8, k = 8 kc + 2 (i % 4)
              const uint32_t r = (i >> 2) & 7u, k = (i >> 5) * 8 + 2 * (i & 3u);
              uint32_t v = 0;
              if (rank == 0 && r < 2) {
                const float w0 = __ldg(wsrc + r * kHidden + k), w1 = __ldg(wsrc + r * kHidden + k + 1);
                v = PREC == 0 ? (uint32_t)__half_as_ushort(__float2half_rn(w0)) |
                                    ((uint32_t)__half_as_ushort(__float2half_rn(w1)) << 16)
                              : (uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(w0)) |
                                    ((uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(w1)) << 16);
              }
              wblk[i] = v;
            }
            ptx::fence_proxy_async_smem();  // read by the output MMA (after the HDONE arrive)
            wcur = ti.model;
          }
          float p[4] = {0.0f, 0.0f, 0.0f, 0.0f};  // CUDA-core share of the output layer
          constexpr uint32_t JT = kOtcKs / 2;     // chunks (of this warp) on the tensor cores
          // this group's leader-CTA poller: wait until both CTAs' groups packed H, then issue
          // the output layer (A = the packed H in place, D = kOtcDCol)
          auto issue_out = [&]() {
            ptx::mbar_wait(bar(B_HDONE + b), (hd_phase >> b) & 1);
            LAKE_TEV(T_OHDONE, it, b, 0);
            ptx::tc_fence_after();
            const bool issuer = lane == 0;
            const uint32_t tm = __shfl_sync(0xffffffffu, tmem, 0);
            const uint32_t idesc_out = ptx::umma_idesc_f16(PREC, 256, 16);
            const uint64_t wd = ptx::umma_desc(sbase + L.wout + gy * kWoutBytes, kLboR8, 1024);
            const uint32_t acc = tm + b * 256;
#pragma unroll
            for (uint32_t ks = 0; ks < kOtcKs; ++ks)
              if (issuer)
                ptx::mma_cg2_ts<PREC>(acc + kOtcDCol, acc + otc_a_col(ks),
                                      wd + ks * ((2 * kLboR8) >> 4), idesc_out, ks);
            if (issuer) ptx::mma_commit_cg2(bar(B_DOUT + b), 0x3);
            __syncwarp();
            LAKE_TEV(T_OCOMMIT, it, b, 0);
          };
#pragma unroll kEpiUnroll
          for (uint32_t j = 0; j < kWarpChunks; ++j) {
            const uint32_t col0 = col_of(j);
            if (j + 1 < kWarpChunks) {
              if (j & 1) ptx::tmem_ld_cols<W>(tbase + col_of(j + 1), ra);
              else ptx::tmem_ld_cols<W>(tbase + col_of(j + 1), rb);
            }
            if (j < JT) {
              // K-steps 2j, 2j+1 on the tensor cores, packed where otc_a_col says. With all
              // 16 there: the last K-step (chunk 7, second half) lands in K-step 13's free
              // half, which this warp read in chunk 6; columns 240..255 stay free for the
              // output MMA. With fewer: chunks 0 and 1 packed shifted (see kOtcDCol)
              const uint32_t dst = kOtcKs == 16 ? ((j == kWarpChunks - 1 && hh == 1) ? kOutLastA : col0)
                                                : ((j < 2 && hh == 0) ? col0 + 8 : col0);
              if (j & 1) epi_to_h_tmem<PREC, W>(rb, hbias, dst, tbase);
              else epi_to_h_tmem<PREC, W>(ra, hbias, dst, tbase);
            } else {
              // on the CUDA cores (fp32; the staged last-layer bias is zero: b0 came from the
              // MMA), after this warp's HDONE arrive: the output MMAs neither read nor write
              // these columns
              if (j & 1) epi_to_logits<PREC, W>(rb, prm, wo, col0, p);
              else epi_to_logits<PREC, W>(ra, prm, wo, col0, p);
            }
            if (j + 1 == JT) {
              ptx::tmem_st_wait();
              ptx::tc_fence_before();
              __syncwarp();
              if (lane == 0) ptx::mbar_arrive_cluster(hdone_leader0 + b * 8);
              LAKE_TEV(T_EHDONE, it, b, warp);
              if (rank == 0 && lw == 1) issue_out();
            }
            if (j + 1 < kWarpChunks) ptx::tmem_ld_wait();
          }
          float p0 = p[0] + p[2], p1 = p[1] + p[3];
          if (kOtcKs < 16 && hh > 0) {  // partials of the quadrant's second warp (read below,
            float *rd = red + row * 2;     // after the group barrier that follows DOUT)
            rd[0] = p0;
            rd[1] = p1;
          }
          hd_phase ^= (1u << b);
          if (lw == 1) ptx::mbar_wait(bar(B_DOUT + b), (do_phase >> b) & 1);
          ptx::named_bar_sync(2 + gy, NG);
          LAKE_TEV(T_EDOUT, it, b, warp);
          do_phase ^= (1u << b);
          ptx::tc_fence_after();
          uint32_t o[2] = {0u, 0u};
          if (hh == 0) {
            ptx::tmem_ld_32x32b_x2(tbase + kOtcDCol, o);
            ptx::tmem_ld_wait();
          }
          ptx::tc_fence_before();
          __syncwarp();
          release_acc(b);
          LAKE_TEV(T_ETEMPTY, it, b, warp);
          const int64_t io = ts.perm ? (int64_t)(int32_t)ptx::opaque_u32(io_ld) : pp;
          if (hh == 0 && pos < ti.count) {
            if (kOtcKs < 16) {
              p0 += red[row * 2 + 0];  // the quadrant's second warp (written before the barrier)
              p1 += red[row * 2 + 1];
            }
            // tensor-core share + this warp's + the second warp's CUDA-core shares + b_out
            const float l0 = (kOtcKs < 16 ? __uint_as_float(o[0]) + p0 : __uint_as_float(o[0])) + wo[2 * kHidden + 0];
            const float l1 = (kOtcKs < 16 ? __uint_as_float(o[1]) + p1 : __uint_as_float(o[1])) + wo[2 * kHidden + 1];
            if (logits) {
              logits[io * 2 + 0] = l0;
              logits[io * 2 + 1] = l1;
            }
            decisions[io] = (l1 > l0) ? 1 : 0;
          }
        } else {
          // last hidden layer: fold the 2-neuron output layer (fp32, CUDA cores). The row's
          // output index is loaded first: with model-grouped staged inputs nothing else has
          // touched perm, so its (DRAM) latency would otherwise sit between the last TMEM
          // read and the accumulator release.
          const int pos = (int)(rank * 128 + row);
          const int64_t pp = ti.begin + pos;
          const int64_t io = (ts.perm && pos < ti.count) ? (int64_t)__ldg(ts.perm + pp) : pp;
          float p[4] = {0.0f, 0.0f, 0.0f, 0.0f};
          const bool hsplit = kL2Split && PREC != 2 && nh >= 2;  // columns 128.. land later
#pragma unroll kEpiUnroll
          for (uint32_t j = 0; j < kWarpChunks; ++j) {
            const uint32_t col0 = col_of(j);
            if constexpr (kPrefetch) {
              const bool mid = hsplit && j + 1 == kWarpChunks / 2;  // next chunk: 2nd half
              if (j + 1 < kWarpChunks && !mid) {
                if (j & 1) ptx::tmem_ld_cols<W>(tbase + col_of(j + 1), ra);
                else ptx::tmem_ld_cols<W>(tbase + col_of(j + 1), rb);
              }
              if (j & 1) EPI_L(rb);
              else EPI_L(ra);
              if (mid) {
                // second half of the last layer: wait for the whole accumulator, then load
                if (lw == 1) ptx::mbar_wait(bar(B_DFULLX + b), (dx_phase >> b) & 1);
                ptx::named_bar_sync(2 + gy, NG);
                dx_phase ^= (1u << b);
                ptx::tc_fence_after();
                if (j & 1) ptx::tmem_ld_cols<W>(tbase + col_of(j + 1), ra);
                else ptx::tmem_ld_cols<W>(tbase + col_of(j + 1), rb);
              }
              if (j + 1 < kWarpChunks) ptx::tmem_ld_wait();
            } else {
              if (j > 0) {
                ptx::tmem_ld_cols<W>(tbase + col0, ra);
                ptx::tmem_ld_wait();
              }
              EPI_L(ra);
            }
          }
#undef EPI_L
          // accumulator b fully read: release it before the reduction and the output stores
          ptx::tc_fence_before();
          __syncwarp();
          release_acc(b);
          float p0 = p[0] + p[2], p1 = p[1] + p[3];
          // combine the kEpiPerQ warps of this quadrant (slices hh = 1.. write partials)
          if (hh > 0) {
            float *rd = red + ((hh - 1) * 128 + row) * 2;
            rd[0] = p0;
            rd[1] = p1;
          }
          ptx::named_bar_sync(red_bar, 32 * kEpiPerQ);
          if (hh == 0) {
#pragma unroll
            for (uint32_t j = 0; j + 1 < kEpiPerQ; ++j) {
              p0 += red[(j * 128 + row) * 2 + 0];
              p1 += red[(j * 128 + row) * 2 + 1];
            }
          }
          // close the exchange before the partial sums are overwritten by the next tile
          // (single group: only NN lacks a later ordering point)
          if (kEpiGroups == 2 || nh == 1) ptx::named_bar_sync(red_bar, 32 * kEpiPerQ);
          if (hh == 0) {
            const float l0 = p0 + wo[2 * kHidden + 0];
            const float l1 = p1 + wo[2 * kHidden + 1];
            if (pos < ti.count) {
              if (logits) {
                logits[io * 2 + 0] = l0;
                logits[io * 2 + 1] = l1;
              }
              decisions[io] = (l1 > l0) ? 1 : 0;
            }
          }
        }
#undef EPI_H
        if (!last) {  // accumulator b fully read by this warp (the last layer released it above)
          ptx::tc_fence_before();
          __syncwarp();
          release_acc(b);
        }
        LAKE_TEV(T_LAYER_END, it, l, warp);
      }
    }
  }

  __syncwarp();  // reconverge role lanes before the .aligned cluster barrier
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == kWarpLoad) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_cg2(tmem, 512);
  }
#if defined(LAKE_TRACE) && defined(LAKE_TRACE_SMEM)
  // each CTA of cluster 0 copies the streams it recorded (rank 1 only records in
  // LAKE_TRACE_DIG / LAKE_TRACE_PAIR builds)
  if (PREC != 2 && tr_buf && cid == 0)
    for (uint32_t i = threadIdx.x; i < 4 * LAKE_TRACE_CAP * 2; i += blockDim.x) {
      const unsigned long long v = reinterpret_cast<const unsigned long long *>(smem + L.total)[i];
      const uint32_t st = i / (LAKE_TRACE_CAP * 2);
#if defined(LAKE_TRACE_DIG)
      const bool mine = rank == 1 ? st == 2 : st != 2;
#elif defined(LAKE_TRACE_PAIR)
      const bool mine = rank == 1 ? st == 2 : st != 2;
#else
      const bool mine = rank == 0;
#endif
      if (mine) tr_buf[i] = v;
    }
#endif
}

template <int PREC, int IN_KIND, bool OTC>
cudaError_t launch_t(const void *in, const TileSched &ts, int nh_layout, uint8_t *dec,
                     float *logits, cudaStream_t s, int grid) {
  const Layout L = tc_layout(nh_layout, PREC);
#if defined(LAKE_TRACE) && defined(LAKE_TRACE_SMEM)
  constexpr uint32_t kTraceBytes = PREC == 2 ? 0u : 4u * LAKE_TRACE_CAP * 16u;
#else
  constexpr uint32_t kTraceBytes = 0;
#endif
  // per-device "attribute set" flags; a race only repeats the (idempotent) attribute call
  static std::atomic<bool> attr_set[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (!attr_set[dev & 63].load(std::memory_order_acquire)) {
    const uint32_t most = OTC ? tc_layout(1, PREC).total : tc_layout(kMaxHiddenLayers, PREC).total;
    cudaError_t e = cudaFuncSetAttribute(mlp_tc_kernel<PREC, IN_KIND, OTC>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)(most + kTraceBytes));
    if (e != cudaSuccess) return e;
    attr_set[dev & 63].store(true, std::memory_order_release);
  }
  mlp_tc_kernel<PREC, IN_KIND, OTC><<<grid, threads_of<OTC>(), L.total + kTraceBytes, s>>>(in, ts, nh_layout,
                                                                                 dec, logits);
  return cudaGetLastError();
}

template <int PREC, int IN_KIND>
cudaError_t launch_o(const void *in, const TileSched &ts, int nh_layout, uint8_t *dec,
                     float *logits, cudaStream_t s, int grid) {
  if constexpr (out_on_tc(1, PREC))
    if (out_on_tc(nh_layout, PREC))
      return launch_t<PREC, IN_KIND, true>(in, ts, nh_layout, dec, logits, s, grid);
  return launch_t<PREC, IN_KIND, false>(in, ts, nh_layout, dec, logits, s, grid);
}

template <int PREC>
cudaError_t launch_p(const void *in, int in_kind, const TileSched &ts, int nh, uint8_t *dec,
                     float *logits, cudaStream_t s, int grid) {
  return in_kind == LAKE_IN_RAW ? launch_o<PREC, LAKE_IN_RAW>(in, ts, nh, dec, logits, s, grid)
                                : launch_o<PREC, LAKE_IN_DIGITS>(in, ts, nh, dec, logits, s, grid);
}

}  // namespace

size_t tc_smem_bytes(int nh_layout, int prec) { return tc_layout(nh_layout, prec).total; }

#ifdef LAKE_TRACE
extern "C" int lake_trace_set(void *dev_buf) {
  return (int)cudaMemcpyToSymbol(g_lake_trace, &dev_buf, sizeof(void *));
}
#endif

cudaError_t launch_mlp_tc(const void *in, int in_kind, int prec, const TileSched &ts, int nh,
                          uint8_t *decisions, float *logits, cudaStream_t s, int device) {
  static std::atomic<int> sms_cache[64];
  int sms = sms_cache[device & 63].load(std::memory_order_relaxed);
  if (!sms) {
    cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    if (e != cudaSuccess) return e;
    sms_cache[device & 63].store(sms, std::memory_order_relaxed);
  }
  const int64_t max_clusters = sms / 2;
  const int64_t clusters = ts.n_tiles < max_clusters ? ts.n_tiles : max_clusters;
  if (clusters <= 0) return cudaSuccess;
  const int grid = (int)(clusters * 2);
  if (nh < 1 || nh > kMaxHiddenLayers) return cudaErrorInvalidValue;
  TileSched t2 = ts;
  t2.nh_cap = nh;
  cudaError_t e;
  if (prec == 0) e = launch_p<0>(in, in_kind, t2, nh, decisions, logits, s, grid);
  else if (prec == 1) e = launch_p<1>(in, in_kind, t2, nh, decisions, logits, s, grid);
  else e = launch_p<2>(in, in_kind, t2, nh, decisions, logits, s, grid);
  count_launch();
  return e;
}

}  // namespace lake
