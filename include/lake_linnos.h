/*
 * lake_linnos.h — C ABI of the B200-native batched LinnOS I/O-latency classifier.
 *
 * The operation is the accelerated hot path of LAKE (Fingler et al., ASPLOS '23):
 * per-I/O features -> decimal digits -> small MLP -> fast/slow decision.
 * Citations are to /root/reference/PAPER.md as "P:<line>" (section named alongside).
 *
 *   - what is classified: "a feature vector that includes the number of pending I/Os
 *     and the completion latency of a fixed number of previous I/Os" (§5.5);
 *     "number of pending I/Os and latency of most recently served I/Os" (§7.1)
 *   - history arrays: "the entry at index 0 is the most recent sample" (§5.2)
 *   - the network: "two layers with 256 and 2 neurons" plus the +1 / +2 variants
 *     "[256,256,2]" and "[256,256,256,2]" (§7.1)
 *   - the calls mirror the feature-registry API (Table 1):
 *     load_model -> lake_linnos_load_weights;
 *     score_features(name, sys, fvs, num) "run inference on a batch, return batch
 *     results" -> lake_linnos_infer / lake_linnos_infer_multi;
 *     one registry (so one model) per block device (Fig. 4 caption) -> model_id.
 *   - "Errors ... are forwarded to the application, which must do its own error
 *     checking" (§4.1) -> every call returns a status; the library never
 *     aborts, prints or throws.
 *
 * Readings of points the paper leaves silent (input width 31, digit widths, saturation,
 * field order, ReLU, biases, FP32 operation order, tie-break) are listed in DESIGN.md §3
 * and SURVEY.md §8(c) S1-S24; the binding ones are restated at each declaration.
 *
 * Conventions for every function below:
 *   - Return value: LAKE_OK (0) or one LAKE_ERR_* code.
 *   - Argument errors are detected on the host before any launch; on error nothing is
 *     written to any output buffer.
 *   - Device: the calling host thread's current CUDA device (cudaSetDevice /
 *     torch.cuda.set_device). `stream` is a cudaStream_t passed as void* and must belong to
 *     that device; NULL means the legacy default stream.
 *   - Asynchrony: lake_linnos_digitize / _infer* only enqueue work on `stream`; they never
 *     synchronise the host. load/unload are synchronous. Loading or unloading a model must
 *     not race with an in-flight infer that uses it.
 *   - Ownership: the caller owns every input/output/workspace buffer. The library owns the
 *     device copies of the weights it makes at load time, until unload.
 *   - Determinism: results are bit-identical run to run and independent of batch
 *     composition and of how a batch is split across calls or GPUs.
 */
#ifndef LAKE_LINNOS_H
#define LAKE_LINNOS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* One raw I/O record, 36 bytes, little endian, no padding (AoS, 4-byte aligned).
 *   q_now     : pending I/Os on the device at issue, including this I/O (Fig. 4
 *               increments pend_ios before committing the vector).
 *   lat_us[k] : completion latency in microseconds of the k-th most recently completed
 *               I/O, k=0 most recent (schema history idiom).
 *   q_hist[k] : that same completed I/O's own q_now at its issue.
 * Values are digitised with saturation, so any uint32 is valid input. */
typedef struct lake_io_raw {
    uint32_t q_now;
    uint32_t lat_us[4];
    uint32_t q_hist[4];
} lake_io_raw_t;

/* Digits layout (LAKE_IN_DIGITS input and lake_linnos_digitize output): uint8_t[n][32].
 * Bytes 0..30 are the 31 input digits, byte 31 is a zero pad:
 *   [0..2]   D3(q_now)
 *   [3..18]  D4(lat_us[0]) D4(lat_us[1]) D4(lat_us[2]) D4(lat_us[3])
 *   [19..30] D3(q_hist[0]) D3(q_hist[1]) D3(q_hist[2]) D3(q_hist[3])
 * Dw(v) = the w decimal digits of min(v, 10^w - 1), most significant first. */
#define LAKE_DIGITS_PER_IO 32
#define LAKE_NUM_INPUTS    31
#define LAKE_HIDDEN        256
#define LAKE_NUM_CLASSES   2

enum lake_status {
    LAKE_OK              = 0,
    LAKE_ERR_INVAL       = 1, /* bad argument: NULL pointer, n < 0, bad flags/arch, bad size */
    LAKE_ERR_NOMODEL     = 2, /* model_id not loaded on the current device                 */
    LAKE_ERR_CUDA        = 3, /* a CUDA runtime call or a kernel launch failed             */
    LAKE_ERR_NOMEM       = 4, /* device allocation failed, or workspace too small          */
    LAKE_ERR_UNSUPPORTED = 5  /* valid request this build does not implement (see flags)   */
};

/* Architectures (§7.1). Hidden layers are 256 wide with ReLU; the output
 * layer has 2 neurons with identity activation; every layer has a bias. */
enum lake_arch {
    LAKE_ARCH_NN  = 0, /* 31 -> 256 -> 2                */
    LAKE_ARCH_NN1 = 1, /* 31 -> 256 -> 256 -> 2         */
    LAKE_ARCH_NN2 = 2  /* 31 -> 256 -> 256 -> 256 -> 2  */
};

/* flags for lake_linnos_infer*: bit 0 = input kind, bits 4..6 = precision path, bits 8..9 =
 * element type of the per-I/O model ids (infer_multi / infer_host; ignored by calls that
 * take no ids). Narrow ids cut the host->device bytes of the host-buffer path (PCIe-bound,
 * DESIGN.md §7): 64 per-SSD models fit in one byte. An id the type cannot hold a loaded model
 * for is simply unknown (decision 0, NaN logits). */
enum lake_flags {
    LAKE_IN_DIGITS  = 0x00, /* in = const uint8_t[n][32]: digits 0..9 (bytes 0..30; the
                               tensor-core multi-model path packs them into 4-bit fields)
                               and a pad byte that is ignored                              */
    LAKE_IN_RAW     = 0x01, /* in = const lake_io_raw_t[n]; digitised inside the kernel  */
    LAKE_PREC_FP32  = 0x00, /* CUDA-core FP32, strict operation order: bit-exact with the
                               oracle (DESIGN.md §3 reading R15)                           */
    LAKE_PREC_F16   = 0x10, /* tcgen05 tensor cores, fp16 operands, fp32 accumulation;
                               NN (one hidden layer) also runs its 2-wide output layer on
                               the tensor cores (fp16 H and W_out), NN+1 / NN+2 in fp32 on
                               CUDA cores; an NN I/O gets the same bits in single- and
                               multi-model calls                         */
    LAKE_PREC_BF16  = 0x20, /* tcgen05 tensor cores, bf16 operands, fp32 accumulation;
                               8 mantissa bits: reported, below the north_star agreement
                               bar on the synthetic models                  */
    LAKE_PREC_TF32  = 0x30, /* tcgen05 tensor cores (kind::tf32), tf32 operands (fp32
                               rounded to 10 mantissa bits), fp32 accumulation, half the
                               fp16 tensor rate; NN+2 streams its last hidden layer's
                               weights from L2 each tile (272 KB/CTA > SMEM) */
    LAKE_PREC_AUTO  = 0x70, /* FP32 below the model's AUTO threshold, else F16 (below)   */
    LAKE_IDS_I32    = 0x000, /* model_ids: int32_t[n] (default)                         */
    LAKE_IDS_U16    = 0x100, /* model_ids: uint16_t[n]                                   */
    LAKE_IDS_U8     = 0x200, /* model_ids: uint8_t[n]                                    */
    LAKE_IN_MASK    = 0x01,
    LAKE_PREC_MASK  = 0x70,
    LAKE_IDS_MASK   = 0x300
};
/* LAKE_PREC_AUTO (the paper's profitability policy, §4.2 P:583-603 and
 * Fig. 3, restricted to GPU paths since there is no CPU fallback): a call with n
 * I/Os takes the bit-exact FP32 path when n < threshold(arch), else the fp16 tensor-core
 * path. Defaults come from the measured C2 curves (profiles/*_sweep_c2.jsonl): the tensor
 * path is chosen where it is at least 20% faster end to end than FP32 — for NN never
 * within the 1..4096 sweep (threshold 8192), for NN+1 and NN+2 from one I/O on. */
#define LAKE_AUTO_TC_MIN_N_NN  8192
#define LAKE_AUTO_TC_MIN_N_NN1 1
#define LAKE_AUTO_TC_MIN_N_NN2 1

#define LAKE_MAX_MODELS 1024   /* model_id range: [0, LAKE_MAX_MODELS) per device */

/* Exact weights-blob length in floats for `arch`, or 0 for an unknown arch:
 * NN 8706, NN+1 74498, NN+2 140290. */
size_t lake_linnos_blob_floats(int32_t arch);

/* load_model (Table 1) + register_classifier(arch=GPU).
 * blob: HOST pointer to fp32 little-endian weights in forward layer order; each layer is
 *   W_l row-major [out][in] followed by b_l[out]:
 *     W0[256][31] b0[256]  (W1[256][256] b1[256])  (W2[256][256] b2[256])  Wout[2][256] bout[2]
 * n_floats must equal lake_linnos_blob_floats(arch), else LAKE_ERR_INVAL.
 * device: CUDA ordinal the model is loaded on (the current device is restored on return).
 * Replaces any model already loaded under (model_id, device). Synchronous with respect to
 * the host (no device-wide synchronisation: the caller must not load/unload a model that an
 * in-flight infer uses). The library deep-copies the blob into device-resident FP32 / fp16 /
 * bf16 images it owns. */
int lake_linnos_load_weights(int32_t model_id, int32_t arch, const float *blob,
                             size_t n_floats, int32_t device);

/* delete_model (Table 1). LAKE_ERR_NOMODEL if nothing is loaded. Synchronous. */
int lake_linnos_unload(int32_t model_id, int32_t device);

/* Architecture of a loaded model through *arch_out; LAKE_ERR_NOMODEL if not loaded. */
int lake_linnos_model_arch(int32_t model_id, int32_t device, int32_t *arch_out);

/* Read / override the AUTO threshold of an architecture (process-wide). Setting returns
 * LAKE_ERR_INVAL for an unknown arch or n_min < 0. */
int lake_linnos_auto_threshold(int32_t arch, int64_t *n_min_out);
int lake_linnos_set_auto_threshold(int32_t arch, int64_t n_min);

/* Digitisation kernel (integer, bit-exact). raw: device lake_io_raw_t[n];
 * digits: device uint8_t[n][32], layout above. n == 0 is a no-op. */
int lake_linnos_digitize(const lake_io_raw_t *raw, int64_t n, uint8_t *digits, void *stream);

/* score_features (Table 1) for one model (one block device).
 *   in        : device input, kind chosen by flags & LAKE_IN_MASK.
 *   decisions : device uint8_t[n]; 1 = slow, 0 = fast. decision = logit[1] > logit[0]
 *               (ties and NaN -> 0).
 *   logits    : device float[n][2] or NULL (not written).
 * Fused: digitise (RAW input) -> every layer -> argmax in one kernel. Tensor-core paths
 * bulk-copy each tile's contiguous input rows (16-B aligned input; otherwise per-row loads).
 * FP32 with n <= 64 (NN: <= 8) runs on one 8-CTA cluster (same strict-order arithmetic).
 * Never allocates; capturable in a CUDA graph. */
int lake_linnos_infer(const void *in, uint32_t flags, int64_t n, int32_t model_id,
                      uint8_t *decisions, float *logits, void *stream);

/* Bytes of device workspace lake_linnos_infer_multi needs for n I/Os. */
size_t lake_linnos_workspace_bytes(int64_t n);

/* Batch scoring across several per-device models in one call (one registry per block
 * device): I/O i is scored with model model_ids[i] (device array of n elements
 * of the type flags & LAKE_IDS_MASK selects: int32_t by default, uint16_t, uint8_t).
 * Groups I/Os by model on the device (histogram, scan, scatter of indices; the order inside
 * a model's group is not preserved and does not affect any result; tensor-core paths also
 * write each I/O's digits as a 16-byte packed row at its grouped position; with 16-B
 * aligned raw records and ids that pass streams them through shared memory with bulk
 * copies, otherwise it loads them per warp - same results either way), then
 * runs the fused kernel over model-homogeneous tiles and scatters results back to the
 * caller's order. Results equal per-model lake_linnos_infer calls bit for bit.
 * workspace: device buffer of at least lake_linnos_workspace_bytes(n) bytes (else
 * LAKE_ERR_NOMEM). A model_id that is out of range or not loaded yields decision 0 and
 * NaN logits for that I/O (device-side ids cannot be checked on the host without a sync);
 * call lake_linnos_multi_status afterwards to read the count of such I/Os. */
int lake_linnos_infer_multi(const void *in, uint32_t flags, int64_t n,
                            const int32_t *model_ids, uint8_t *decisions, float *logits,
                            void *workspace, size_t ws_bytes, void *stream);

/* The two halves of lake_linnos_infer_multi, exposed so a caller can time the fused MLP
 * kernel on its own: _group builds the model grouping in `workspace`; _grouped runs the
 * fused kernel on that grouping. _group followed by _grouped == _infer_multi. */
int lake_linnos_multi_group(int64_t n, const int32_t *model_ids, void *workspace,
                            size_t ws_bytes, void *stream);
int lake_linnos_multi_grouped(const void *in, uint32_t flags, int64_t n, uint8_t *decisions,
                              float *logits, void *workspace, size_t ws_bytes, void *stream);

/* Synchronous: number of I/Os in the last _group on this workspace whose model_id was
 * unknown (out of range or not loaded). */
int lake_linnos_multi_status(const void *workspace, size_t ws_bytes, int64_t *n_unknown,
                             void *stream);

/* End-to-end call with HOST buffers (the latency path of Fig. 8, "including data copying
 * latencies"): h_in (pinned host memory recommended, else the copies are
 * synchronous) is processed in chunks of up to 2^20 I/Os through a 3-stage pipeline:
 * host->device copy on an internal stream, lake_linnos_infer_multi (h_model_ids != NULL) or
 * lake_linnos_infer(model_id) on `stream`, device->host copy of decisions (and logits if
 * h_logits != NULL) on a second internal stream, so chunk i+1's upload and chunk i-1's
 * download overlap chunk i's kernels. Synchronous: returns when every output is on the host.
 * d_staging: device buffer of at least lake_linnos_host_staging_bytes(n, flags) bytes (two
 * chunk slots). LAKE_PREC_AUTO is resolved once for the whole batch. Batches of at most
 * 2^14 I/Os whose host buffers are all pinned and mapped (cudaHostAlloc / cudaHostRegister
 * under UVA) skip the copies: the kernel reads and writes host memory directly (zero-copy),
 * which is what bounds small-batch latency (Fig. 8's batch sizes).
 * h_model_ids holds n elements of the type flags & LAKE_IDS_MASK selects (int32_t by
 * default, uint16_t or uint8_t; the pointer type is nominal): the upload is PCIe-bound, so
 * one-byte ids move 37 instead of 40 bytes per I/O. infer_multi reads its device
 * model_ids the same way. */
size_t lake_linnos_host_staging_bytes(int64_t n, uint32_t flags);
int lake_linnos_infer_host(const void *h_in, uint32_t flags, int64_t n, int32_t model_id,
                           const int32_t *h_model_ids, uint8_t *h_decisions, float *h_logits,
                           void *d_staging, size_t staging_bytes, void *stream);

/* GPU feature capture: the raw records the feature registry would
 * capture on issue and completion (Fig. 4 / Fig. 5), computed for a whole trace.
 * Inputs (device pointers, n entries, any order): arrival_ns[i], complete_ns[i] (int64, ns,
 * 0 <= arrival < complete < 2^47) and device[i] (int32 in [0, 65535]; NULL = one device).
 * Output raw_out[i] (lake_io_raw_t, device memory), with DESIGN.md readings R7-R10:
 *   q_now     = I/Os of the same device issued at or before i (ties in arrival by index,
 *               i included) that complete after a_i; an I/O completing exactly at a_i counts
 *               as completed;
 *   history k = the k-th newest completed I/O of the device by (complete_ns, index):
 *               lat_us = floor((complete - arrival) / 1000) (clamped to uint32), q_hist =
 *               its own q_now; zeros when fewer than k+1 have completed.
 * workspace: device buffer of lake_linnos_capture_workspace_bytes(n) bytes (else
 * LAKE_ERR_NOMEM). Asynchronous on `stream`; n <= INT32_MAX. Bit-exact (integer). */
size_t lake_linnos_capture_workspace_bytes(int64_t n);
int lake_linnos_capture(const int64_t *arrival_ns, const int64_t *complete_ns,
                        const int32_t *device, int64_t n, lake_io_raw_t *raw_out,
                        void *workspace, size_t ws_bytes, void *stream);

/* Persistent resident-weights server: the latency path for small
 * batches, against the paper's profitability problem (§4.2; Fig. 8).
 * _server_start launches one kernel that stays resident on an 8-CTA cluster (8 SMs) with a
 * slice of the model's FP32 weights in each CTA's shared memory, and a mailbox in mapped
 * pinned host memory. _server_infer copies up to LAKE_SERVER_MAX_BATCH raw records (HOST
 * pointer) into the mailbox, rings the doorbell (a sequence number the kernel polls with
 * system-scope acquire loads), and spins until the kernel has written the decisions (and
 * logits if non-NULL, HOST pointers) back into the mailbox: no launch, no memcpy, no stream
 * sync per batch. Arithmetic = the FP32 path (bit-exact with the oracle). Calls on one
 * server must not overlap (one batch in flight). The server keeps its own copy of the
 * weights: unloading the model afterwards is safe. _server_stop ends the kernel.
 * Errors: LAKE_ERR_INVAL (n < 0 or > LAKE_SERVER_MAX_BATCH, NULL), LAKE_ERR_NOMODEL,
 * LAKE_ERR_CUDA (the kernel died or never answered). */
#define LAKE_SERVER_MAX_BATCH 64
typedef struct lake_server lake_server_t;
int lake_linnos_server_start(int32_t model_id, lake_server_t **server_out);
int lake_linnos_server_infer(lake_server_t *server, const lake_io_raw_t *h_raw, int32_t n,
                             uint8_t *h_decisions, float *h_logits);
int lake_linnos_server_stop(lake_server_t *server);

/* Number of kernels this library launched on the current device since the last reset
 * (host-side counter; used by the bench to report gpu_launches). */
uint64_t lake_linnos_launch_count(void);
void lake_linnos_reset_launch_count(void);

/* Device-side timing of the fused MLP kernel (the dominant kernel), for the bench's
 * roofline: while enabled, every fused-kernel launch by _infer / _multi_grouped is
 * bracketed by two CUDA events recorded on the launch stream. _profile_read waits for
 * the recorded events, returns the summed elapsed milliseconds and the number of
 * bracketed launches, and resets the accumulator. Enabling also resets it. */
int lake_linnos_profile_enable(int enable);
int lake_linnos_profile_read(double *total_ms, int64_t *n_launches);

/* Static string for a status code; never NULL. */
const char *lake_linnos_strerror(int status);

#ifdef __cplusplus
}
#endif
#endif /* LAKE_LINNOS_H */
