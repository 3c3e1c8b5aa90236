// lake_internal.h — internal types shared by the C-ABI layer (api.cu) and the kernels.
// Not part of the public ABI (include/lake_linnos.h is).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/lake_linnos.h"

namespace lake {

constexpr int kHidden = 256;
constexpr int kInputs = 31;
constexpr int kMaxHiddenLayers = 3;

// ---- FP32 CUDA-core path (mlp_fp32.cu) ------------------------------------------------
// Per layer l the weights are stored transposed, W^T[k][j], k < K_l, with the 256 output
// columns permuted so that thread tc's 8 columns {tc + 32*jj} are two contiguous float4
// groups: position p(j) = (jj/4)*128 + tc*4 + (jj%4) with tc = j%32, jj = j/32.
#ifndef LAKE_F32_RN
#define LAKE_F32_RN 16  // FP32 register tile columns per thread: 16 (M 128, 1 CTA/SM) or 8 (M 64)
#endif
constexpr int kF32TileRN = LAKE_F32_RN;
constexpr int kF32TileM = kF32TileRN == 16 ? 128 : 64;  // I/Os per CTA tile (mlp_fp32.cu)
constexpr int kF32Threads = 256;
#ifndef LAKE_F32_KC
#define LAKE_F32_KC 16  // 2 CTAs per SM fit only with 16-row chunks (64 was best at 1 CTA/SM)
#endif
constexpr int kF32KChunk = LAKE_F32_KC;  // rows of W^T staged per pipeline stage
constexpr int kF32ActStride = 68;   // floats per activation row in SMEM (64 + 4 pad)

// ---- tcgen05 path (mlp_tc.cu) ------------------------------------------------------------
// A CTA pair (cluster of 2, cta_group::2) processes a 256-row tile: each CTA owns 128 rows
// of A and D, and holds half (N/2 rows) of every weight matrix, in the K-major SWIZZLE_NONE
// UMMA layout: core matrix (8 rows x 16 B) for (row group rg, k group kg) at byte offset
// kg * (R * 16) + rg * 128, i.e. LBO = R*16 bytes (K direction), SBO = 128 bytes.
constexpr int kTcRowsPerCta = 128;
constexpr int kTcTileRows = 256;
constexpr int kTcK0 = 32;                                   // 31 digits + zero pad
// Operand element size per precision: prec 0 fp16, 1 bf16 (2 B), 2 tf32 (4 B, fp32 bits
// with the low 13 mantissa bits zero). A core matrix is 8 rows x 16 B in every case.
__host__ __device__ constexpr uint32_t tc_elem_bytes(int prec) { return prec == 2 ? 4u : 2u; }
__host__ __device__ constexpr uint32_t tc_w0_half_bytes(int prec) {
  return 128u * kTcK0 * tc_elem_bytes(prec);        // 8 KB (16-bit) / 16 KB (tf32)
}
__host__ __device__ constexpr uint32_t tc_wh_half_bytes(int prec) {
  return 128u * kHidden * tc_elem_bytes(prec);      // 64 KB / 128 KB
}
constexpr uint32_t kTcW0HalfBytes = tc_w0_half_bytes(0);
constexpr uint32_t kTcWhHalfBytes = tc_wh_half_bytes(0);
// fp16/bf16: each hidden layer l >= 1 is followed by a bias block, 128 rows x K 16 in the
// operand layout with b_l in K column 0 (zeros elsewhere): one extra MMA with a constant
// "ones" A tile initialises the accumulator with the bias, so no epilogue adds a bias
// (layer 0's bias rides in W0's K slot 31). tf32 has no SMEM for the blocks (0 bytes).
__host__ __device__ constexpr uint32_t tc_bias_block_bytes(int prec) {
  return prec == 2 ? 0u : 128u * 16u * tc_elem_bytes(prec);  // 4 KB
}
// stride between hidden layers in the image, and a hidden layer's offset
__host__ __device__ constexpr uint32_t tc_layer_stride(int prec) {
  return tc_wh_half_bytes(prec) + tc_bias_block_bytes(prec);
}
__host__ __device__ constexpr uint32_t tc_wh_off(int l, int prec) {
  return tc_w0_half_bytes(prec) + (l - 1) * tc_layer_stride(prec);
}
// Per-rank weight image: W0 half | hidden-layer halves (+ bias blocks). The fp32 biases and
// the 2-wide output layer are staged by the epilogue from the FP32 image (b[0] .. b[nh-1],
// W_out[2][256], b_out[2] are contiguous there).
__host__ __device__ constexpr uint32_t tc_image_bytes(int nh, int prec = 0) {
  return tc_w0_half_bytes(prec) + (nh - 1) * tc_layer_stride(prec);
}
// Bytes of the per-rank image kept resident in SMEM. Everything, except for tf32 NN+2
// (272 KB per rank > 227 KB): its last hidden layer (W2, 128 KB per rank) is streamed
// from L2 through an SMEM ring, K-chunk by K-chunk, every tile.
__host__ __device__ constexpr uint32_t tc_resident_bytes(int nh, int prec) {
  return (prec == 2 && nh == 3) ? tc_image_bytes(2, 2) : tc_image_bytes(nh, prec);
}
// Layer-0 K order of the tensor-core path (the MMA's reduction order is free, so W0's columns
// are permuted to match): slot -> canonical digit index. Slots 0-15 are the four
// 4-digit latency fields, 16-25 the last two digits ("tails") of the five 3-digit queue
// fields, 26-30 their leading digits ("heads"), 31 the zero pad - so every operand pair of the
// layer-0 A row is one table lookup (tc digitiser) or one byte of the packed row (nibbles).
__host__ __device__ constexpr int tc_slot_digit(int s) {
  return s < 16 ? 3 + s                                   // lat0..lat3: canonical 3..18
       : s < 26 ? ((s - 16) / 2 == 0 ? 1 : 17 + 3 * ((s - 16) / 2)) + (s & 1)  // tails
       : s < 31 ? ((s - 26) == 0 ? 0 : 16 + 3 * (s - 26))   // heads: 0, 19, 22, 25, 28
       : 31;                                                // pad
}
static_assert(tc_slot_digit(16) == 1 && tc_slot_digit(17) == 2 && tc_slot_digit(18) == 20 &&
              tc_slot_digit(25) == 30 && tc_slot_digit(26) == 0 && tc_slot_digit(27) == 19 &&
              tc_slot_digit(30) == 28 && tc_slot_digit(15) == 18, "tc slot permutation");
constexpr uint32_t kTcRingSlotBytes = 8192;  // tf32 W2 ring slot: 128 rows x K 16
constexpr uint32_t kTcRingSlots = 4;

struct DevModel {
  int32_t arch;      // -1 = slot empty
  int32_t nh;        // hidden layers: 1, 2, 3
  // tcgen05 images: [0]=fp16, [1]=bf16, [2]=tf32; each holds rank-0 half then rank-1 half
  // (tc_image_bytes(nh, prec) bytes per rank half).
  const uint8_t *tc_img[3];
  // FP32 path
  const float *wt[kMaxHiddenLayers];  // permuted W^T; layer 0 is [32][256] (row 31 zero)
  const float *b[kMaxHiddenLayers];
  const float *wout;                  // [2][256]
  const float *bout;                  // [2]
  // cluster image (server.cu: persistent server and FP32 small-batch kernel): per cluster
  // rank r < 8, kServerRankFloats floats: b[3][32] | W_out[2][256] | b_out[4] | W0^T[31][32]
  // | W_l^T[2][256][32], the rank's 32 output columns of every hidden layer
  const float *srv;
};
constexpr int kServerCtas = 8;
constexpr int kServerSlice = kHidden / kServerCtas;
constexpr uint32_t kServerRankFloats = kMaxHiddenLayers * kServerSlice + 2 * kHidden + 4 +
                                       kInputs * kServerSlice +
                                       (kMaxHiddenLayers - 1) * kHidden * kServerSlice;
// bytes of a rank's block a model with nh hidden layers uses (a prefix; multiple of 16)
__host__ __device__ constexpr uint32_t server_block_bytes(int nh) {
  return 4u * (kMaxHiddenLayers * kServerSlice + 2 * kHidden + 4 + kInputs * kServerSlice +
               (nh - 1) * kHidden * kServerSlice);
}
static_assert(server_block_bytes(1) % 16 == 0 && kServerRankFloats % 4 == 0, "bulk copy sizes");

// Tile schedule. Single-model calls use tile_model == nullptr (all tiles -> `model`) and
// implicit contiguous tiles; multi-model calls read a device-built grouping.
struct TileSched {
  const int32_t *tile_model;   // [n_tiles] model slot per tile, or nullptr
  const int64_t *tile_begin;   // [n_tiles] first position in `perm`
  const int32_t *tile_count;   // [n_tiles] rows in the tile
  const int32_t *perm;         // position -> I/O index, or nullptr (identity)
  const uint4 *pdig;           // packed digit rows in position order (multi, TC), or nullptr
  const int32_t *n_tiles_dev;  // device tile count (multi) or nullptr
  int64_t n_tiles;             // host tile count (single) / upper bound (multi)
  int64_t n;                   // I/Os
  const DevModel *table;       // device model table (multi)
  DevModel model;              // single-model copy
  int nh_cap;                  // tcgen05 path: the SMEM layout's hidden-layer count (set at launch)
  const int32_t *tile_split_dev;  // multi (tcgen05): NN tiles are [0, *split), the rest after
  int part;                    // 0: every tile; 1: tiles [0, *split); 2: tiles [*split, n_tiles)
};

// Kernel launchers (return cudaError_t of the launch).
cudaError_t launch_digitize(const lake_io_raw_t *raw, int64_t n, uint8_t *digits,
                            cudaStream_t s);
cudaError_t launch_mlp_fp32(const void *in, int in_kind, const TileSched &ts,
                            uint8_t *decisions, float *logits, cudaStream_t s, int device);
cudaError_t launch_mlp_tc(const void *in, int in_kind, int prec, const TileSched &ts, int nh,
                          uint8_t *decisions, float *logits, cudaStream_t s, int device);
// Stable LSD radix sort of (u64 key, i32 value) pairs over the low `bits` key bits (sort.cu);
// *in_alt: the result is in the _alt buffers (odd number of 8-bit passes).
size_t radix_sort_workspace_bytes(int64_t n);
cudaError_t radix_sort_pairs(uint64_t *keys, uint64_t *keys_alt, int32_t *vals, int32_t *vals_alt,
                             int64_t n, int bits, void *ws, cudaStream_t s, bool *in_alt,
                             const int32_t *d_npasses = nullptr);
// Grouping for infer_multi (group.cu).
size_t group_workspace_bytes(int64_t n);
int64_t group_max_tiles(int64_t n, int tile_rows);
// id_kind: 0 int32, 1 uint16, 2 uint8 (flags bits 8..9)
// in != nullptr: the scatter also writes the packed digit rows of `in` (in_kind) in grouped
// order; otherwise launch_group_pack fills them later by gathering through perm
cudaError_t launch_group(int64_t n, const void *model_ids, int id_kind, const DevModel *table,
                         void *ws, const void *in, int in_kind, cudaStream_t s);
cudaError_t launch_group_pack(void *ws, int64_t n, const void *in, int in_kind, cudaStream_t s);
// which = 0: 64-row FP32 tiles, 1: 256-row tensor-core tiles
void group_sched(void *ws, int64_t n, int which, const DevModel *table, TileSched *ts);
cudaError_t launch_unknown_fill(void *ws, int64_t n, uint8_t *decisions, float *logits,
                                cudaStream_t s);
struct GroupView {
  int32_t *perm;
  int64_t *n_unknown;
  int32_t *counts;
};
GroupView group_view(void *ws, int64_t n);
size_t tc_smem_bytes(int nh_layout, int prec);

// GPU feature capture (capture.cu)
size_t capture_workspace_bytes(int64_t n);
cudaError_t launch_capture(const int64_t *a, const int64_t *c, const int32_t *dev, int64_t n,
                           uint32_t *raw, void *ws, size_t ws_bytes, cudaStream_t s);

// FP32 small-batch kernel (server.cu): one 8-CTA cluster, weights spread over the cluster,
// n <= LAKE_SERVER_MAX_BATCH rows of device input; same strict-order arithmetic (bit-exact)
cudaError_t launch_fp32_small(const DevModel &m, const void *in, int in_kind, int64_t n,
                              uint8_t *dec, float *logits, cudaStream_t s);
// persistent doorbell server (server.cu)
struct Server;
int server_start(const DevModel &m, int device, Server **out);
int server_infer(Server *s, const lake_io_raw_t *raw, int32_t n, uint8_t *dec, float *logits);
int server_stop(Server *s);
size_t server_smem_bytes();
int server_device(const Server *s);

void count_launch(int k = 1);

// deferred.cu: releases that never block behind a running persistent server
void release_device(void *p, int device);  // cudaFree on `device`, now or when no server runs
void release_host(void *p);                 // cudaFreeHost, now or when no server runs
void servers_started();
void servers_stopped();

}  // namespace lake
