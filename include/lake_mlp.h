/*
 * lake_mlp.h — C ABI of the second workload on the fused-MLP family (SURVEY.md §8(f)
 * NEXT-4): small classifier MLPs of the kind LAKE ports for load balancing and for
 * readahead classification.
 *
 *   - MLLB: "MLLB [16] used a multi-layer perceptron for load balancing. We port MLLB's
 *     model to CUDA" (§7.3); GPU profitable "for batches larger than 128
 *     inputs" (Fig. 10).
 *   - KML: "uses a pre-trained neural network to classify applications according to I/O
 *     patterns, where each pattern has an optimal readahead configuration" (§7.4,
 *     P:1493-1496); "We port KML's NN ... to a kernel space module that uses CUDA"
 *     (P:1499-1500); profitable above 64 inputs (Fig. 11).
 *   - batch scoring is the feature registry's score_features (Table 1).
 *
 * PAPER.md gives neither model's layer widths, activation or features, so this ABI takes
 * them as arguments; the shapes the tests and the bench use are readings R25-R28 in
 * DESIGN.md §3 (MLLB 15->10->10->2 ReLU, KML 5->15->15->4 sigmoid).
 *
 * Conventions (status codes, devices, streams, ownership, asynchrony, determinism) are
 * those of include/lake_linnos.h, whose enum lake_status this header reuses:
 *   - every function returns LAKE_OK or a LAKE_ERR_* code and never aborts, prints or
 *     throws; argument errors are found on the host before any launch, and then nothing is
 *     written to any output;
 *   - device pointers belong to the calling thread's current CUDA device; `stream` is a
 *     cudaStream_t passed as void* (NULL = legacy default stream);
 *   - lake_mlp_infer only enqueues work; load / unload are synchronous and must not race
 *     with an in-flight infer of the same model;
 *   - results are bit-identical run to run and independent of batch composition.
 */
#ifndef LAKE_MLP_H
#define LAKE_MLP_H

#include <stddef.h>
#include <stdint.h>

#include "lake_linnos.h"

#ifdef __cplusplus
extern "C" {
#endif

#define LAKE_MLP_MAX_LAYERS 4   /* weight layers (hidden layers + output), 1..4 */
#define LAKE_MLP_MAX_WIDTH 64   /* every width, input included */
#define LAKE_MLP_MAX_MODELS 256 /* model ids 0..255 per device */

/* Hidden-layer activation; the output layer is always the identity. */
enum lake_mlp_act {
    LAKE_ACT_RELU = 0,    /* h = (z > 0.0f) ? z : +0.0f                          (R15) */
    LAKE_ACT_SIGMOID = 1  /* h = 1 / (1 + exp(-z)); computed on the SFU (ex2.approx,
                             rcp.approx): outputs within 1e-5 relative of the binary32
                             definition 1.0f / (1.0f + expf(-z)) (R27)                 */
};

/* Exact blob length in floats for a shape, or 0 if the shape is invalid:
 * sum over layers l of widths[l+1] * widths[l] + widths[l+1]. widths has n_layers + 1
 * entries: widths[0] = input width, widths[n_layers] = C classes (>= 2). */
size_t lake_mlp_blob_floats(int32_t n_layers, const int32_t *widths);

/* load_model + register_classifier(arch = GPU) (Table 1) for one small MLP.
 *   widths : HOST int32[n_layers + 1], each 1..LAKE_MLP_MAX_WIDTH, widths[n_layers] >= 2.
 *   act    : enum lake_mlp_act for every hidden layer.
 *   blob   : HOST fp32, forward layer order, each layer W_l row-major [out][in] then
 *            b_l[out]; n_floats must equal lake_mlp_blob_floats(), every value finite.
 *   device : CUDA ordinal (the current device is restored on return).
 * Replaces a model already loaded under (model_id, device). The library deep-copies the
 * blob into a device image it owns until unload. Errors: LAKE_ERR_INVAL (bad id, shape,
 * act, length, non-finite value, device), LAKE_ERR_NOMEM, LAKE_ERR_CUDA. */
int lake_mlp_load(int32_t model_id, int32_t n_layers, const int32_t *widths, int32_t act,
                  const float *blob, size_t n_floats, int32_t device);

/* delete_model (Table 1). LAKE_ERR_NOMODEL if nothing is loaded. Synchronous. */
int lake_mlp_unload(int32_t model_id, int32_t device);

/* score_features (Table 1): one fused kernel per call, every layer and the argmax
 * on CUDA cores in FP32, in the oracle's operation order (per output: acc from +0.0f,
 * fmaf over inputs in ascending order, + bias, activation), so ReLU models are bit-exact.
 *   x       : device float[n][widths[0]], row-major, 4-byte aligned.
 *   classes : device int32[n]: the first c with out[c] maximal (ties -> lowest index, a NaN
 *             output never wins; for C = 2 this is LinnOS's logit1 > logit0, R14).
 *   out     : device float[n][C] output-layer values, or NULL (not written).
 * n == 0 is a no-op. Errors: LAKE_ERR_INVAL (n < 0, n > INT32_MAX, NULL x / classes,
 * misaligned pointer), LAKE_ERR_NOMODEL (model not loaded on the current device),
 * LAKE_ERR_CUDA (launch failure). */
int lake_mlp_infer(const float *x, int64_t n, int32_t model_id, int32_t *classes, float *out,
                   void *stream);

/* Device staging bytes lake_mlp_infer_host needs for n rows of width_in inputs and
 * `classes` outputs (0 for n < 0 or a width outside 1..LAKE_MLP_MAX_WIDTH). */
size_t lake_mlp_host_staging_bytes(int64_t n, int32_t width_in, int32_t classes);

/* score_features with HOST buffers, synchronous (returns after the results are in host
 * memory): the batch-latency path of Fig. 10 / Fig. 11 ("including data copying"). When
 * every host buffer is pinned and mapped (UVA), the kernel reads the features from and
 * writes the classes / outputs to host memory directly (no copy-engine round trips);
 * otherwise it copies through d_staging (device, >= lake_mlp_host_staging_bytes).
 *   h_x : host float[n][widths[0]]; h_classes : host int32[n]; h_out : host float[n][C]
 *   or NULL. Errors as lake_mlp_infer, plus LAKE_ERR_NOMEM if staging is needed and short. */
int lake_mlp_infer_host(const float *h_x, int64_t n, int32_t model_id, int32_t *h_classes,
                        float *h_out, void *d_staging, size_t staging_bytes, void *stream);

/* Shape of a loaded model: *n_layers_out and widths_out[0..n_layers] (caller provides
 * LAKE_MLP_MAX_LAYERS + 1 entries), *act_out. LAKE_ERR_NOMODEL if not loaded. */
int lake_mlp_model_shape(int32_t model_id, int32_t device, int32_t *n_layers_out,
                         int32_t *widths_out, int32_t *act_out);

/* Kernel selection. Shapes with a compile-time-specialised kernel (the MLLB and KML
 * readings, R25/R26) use it by default; enable != 0 routes every model through the generic
 * runtime-shape kernel instead (process-wide; both kernels compute the same values — the
 * parity tests run both). Returns the previous setting (0 or 1). */
int lake_mlp_force_generic(int32_t enable);

#ifdef __cplusplus
}
#endif

#endif /* LAKE_MLP_H */
