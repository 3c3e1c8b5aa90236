/*
 * lake_oracle.c — CPU ORACLE for the batched LinnOS I/O-latency classifier.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library. The product path
 * (paper_conf_asplos_finglertyshar23_b200/) never imports, links or calls it, and shares
 * no code, header, table or constant generator with it.
 *
 * What it computes is the plain definition (the method is exact, not an approximation),
 * written out in the paper's order. Citations are /root/reference/PAPER.md line numbers.
 *
 *   feature vector: pending I/Os + latencies of a fixed number of previous I/Os
 *                   (§5.5; §7.1); history index 0 = most recent
 *                   (§5.2)
 *   network:        "two layers with 256 and 2 neurons" (+1: [256,256,2],
 *                   +2: [256,256,256,2]) (§7.1)
 *   decision:       classify each I/O "into slow or fast" (§7.1)
 *   batch scoring:  score_features(name, sys, fvs, num) (Table 1; §5.4)
 *
 * Readings where the paper is silent (DESIGN.md §3 / SURVEY.md §8(c)):
 *   R1-R6  31 inputs = D3(q_now) | D4(lat[0..3]) | D3(q_hist[0..3]); Dw(v) = the w decimal
 *          digits of min(v, 10^w-1), most significant first (saturating).
 *   R11    ReLU on hidden layers, identity on the output layer.  R12  biases everywhere.
 *   R13    digit values 0..9 are the float inputs.
 *   R14    decision = (logit[1] > logit[0]) ? 1 : 0  (1 = slow; ties, NaN -> 0).
 *   R15    per output: acc = +0.0f; for k ascending acc = fmaf(h[k], W[j][k], acc);
 *          z = acc + b[j] (one rounding); hidden h'[j] = (z > 0.0f) ? z : 0.0f.
 *
 * Pins (tests/test_oracle_*.py, -m "not gpu"): hand-worked digit examples
 * (tests/golden/digitize_examples.txt), brute-force digit round trip, tiny all-integer
 * MLPs checked exactly against int64 arithmetic, IEEE rounding examples that fix the
 * operation order of R15, ReLU zeroing, argmax symmetry, batch independence, hidden-unit
 * permutation, and the full-size MLP against a numpy float64 GEMM chain.
 *
 * Build: gcc -std=c99 -O2 -mfma -ffp-contract=off -fno-fast-math -fopenmp -shared -fPIC
 * (no FTZ, no contraction: every rounding below is the one written).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_NUM_INPUTS 31
#define ORACLE_RAW_FIELDS 9 /* q_now, lat_us[4], q_hist[4] */

/* Dw(v): the w decimal digits of min(v, 10^w - 1), most significant first (R3-R5). */
static void decimal_digits(uint32_t v, int w, int *out)
{
    uint32_t cap = 1;
    for (int i = 0; i < w; ++i) cap *= 10u;
    cap -= 1u;
    uint32_t m = (v < cap) ? v : cap;
    for (int i = w - 1; i >= 0; --i) {
        out[i] = (int)(m % 10u);
        m /= 10u;
    }
}

/* One record {q_now, lat_us[0..3], q_hist[0..3]} -> 31 digits in field order R6. */
void oracle_digitize_one(const uint32_t *rec, int *digits31)
{
    int pos = 0;
    decimal_digits(rec[0], 3, digits31 + pos);               /* q_now      */
    pos += 3;
    for (int k = 0; k < 4; ++k) {                             /* lat_us[k]  */
        decimal_digits(rec[1 + k], 4, digits31 + pos);
        pos += 4;
    }
    for (int k = 0; k < 4; ++k) {                             /* q_hist[k]  */
        decimal_digits(rec[5 + k], 3, digits31 + pos);
        pos += 3;
    }
}

/* raw: uint32[n][9]; out: uint8[n][31]. */
void oracle_digitize(const uint32_t *raw, int64_t n, uint8_t *out)
{
    for (int64_t i = 0; i < n; ++i) {
        int d[ORACLE_NUM_INPUTS];
        oracle_digitize_one(raw + i * ORACLE_RAW_FIELDS, d);
        for (int j = 0; j < ORACLE_NUM_INPUTS; ++j) out[i * ORACLE_NUM_INPUTS + j] = (uint8_t)d[j];
    }
}

/* One fully connected layer for one I/O, R15 order. W row-major [n_out][n_in]. */
static void dense_layer(const float *h, int n_in, const float *W, const float *b, int n_out,
                        int relu, float *out)
{
    for (int j = 0; j < n_out; ++j) {
        float acc = +0.0f;
        for (int k = 0; k < n_in; ++k) acc = fmaf(h[k], W[(int64_t)j * n_in + k], acc);
        float z = acc + b[j];
        out[j] = relu ? ((z > 0.0f) ? z : 0.0f) : z;
    }
}

/*
 * Generic MLP over n I/Os. widths[0..n_layers]: widths[0] = input width, widths[n_layers]
 * = 2 classes. blob: per layer W_l[widths[l+1]][widths[l]] then b_l[widths[l+1]].
 * x: float[n][widths[0]]; logits: float[n][2]; decisions: uint8[n].
 * The LinnOS architectures are widths {31,256,2}, {31,256,256,2}, {31,256,256,256,2}.
 */
int oracle_mlp(int n_layers, const int *widths, const float *blob, const float *x, int64_t n,
               float *logits, uint8_t *decisions, int nthreads)
{
    if (n_layers < 1 || widths[n_layers] != 2) return 1;
    int maxw = 0;
    for (int l = 0; l <= n_layers; ++l) {
        if (widths[l] <= 0) return 1;
        if (widths[l] > maxw) maxw = widths[l];
    }
#ifdef _OPENMP
    const int nt = nthreads > 0 ? nthreads : omp_get_num_procs();  /* no global OpenMP state */
#else
    (void)nthreads;
#endif
#pragma omp parallel for schedule(static) num_threads(nt)
    for (int64_t i = 0; i < n; ++i) {
        float bufa[maxw], bufb[maxw];            /* C99 VLAs: per-I/O activations */
        float *h = bufa, *hn = bufb;
        memcpy(h, x + i * widths[0], sizeof(float) * (size_t)widths[0]);
        const float *p = blob;
        for (int l = 0; l < n_layers; ++l) {
            const float *W = p;
            const float *b = p + (int64_t)widths[l + 1] * widths[l];
            p = b + widths[l + 1];
            int relu = (l + 1 < n_layers);
            dense_layer(h, widths[l], W, b, widths[l + 1], relu, hn);
            float *t = h; h = hn; hn = t;
        }
        logits[2 * i + 0] = h[0];
        logits[2 * i + 1] = h[1];
        decisions[i] = (h[1] > h[0]) ? 1 : 0;   /* R14 */
    }
    return 0;
}

/* LinnOS arch id (0 = NN, 1 = NN+1, 2 = NN+2) -> layer widths. */
static int linnos_widths(int arch, int *widths)
{
    if (arch < 0 || arch > 2) return -1;
    int n_layers = arch + 2;
    widths[0] = ORACLE_NUM_INPUTS;
    for (int l = 1; l < n_layers; ++l) widths[l] = 256;
    widths[n_layers] = 2;
    return n_layers;
}

/* score_features for one model on raw records: digitise then MLP. */
int oracle_infer_raw(int arch, const float *blob, const uint32_t *raw, int64_t n,
                     float *logits, uint8_t *decisions, int nthreads)
{
    int widths[8];
    int n_layers = linnos_widths(arch, widths);
    if (n_layers < 0) return 1;
    float *x = (float *)malloc(sizeof(float) * (size_t)(n > 0 ? n : 1) * ORACLE_NUM_INPUTS);
    if (!x) return 2;
    for (int64_t i = 0; i < n; ++i) {
        int d[ORACLE_NUM_INPUTS];
        oracle_digitize_one(raw + i * ORACLE_RAW_FIELDS, d);
        for (int j = 0; j < ORACLE_NUM_INPUTS; ++j) x[i * ORACLE_NUM_INPUTS + j] = (float)d[j];
    }
    int rc = oracle_mlp(n_layers, widths, blob, x, n, logits, decisions, nthreads);
    free(x);
    return rc;
}

/* Same, on digits uint8[n][31] (the LAKE_IN_DIGITS input kind without its pad byte). */
int oracle_infer_digits(int arch, const float *blob, const uint8_t *digits31, int64_t n,
                        float *logits, uint8_t *decisions, int nthreads)
{
    int widths[8];
    int n_layers = linnos_widths(arch, widths);
    if (n_layers < 0) return 1;
    float *x = (float *)malloc(sizeof(float) * (size_t)(n > 0 ? n : 1) * ORACLE_NUM_INPUTS);
    if (!x) return 2;
    for (int64_t i = 0; i < n * ORACLE_NUM_INPUTS; ++i) x[i] = (float)digits31[i];
    int rc = oracle_mlp(n_layers, widths, blob, x, n, logits, decisions, nthreads);
    free(x);
    return rc;
}

/*
 * Feature capture (NEXT-1; Fig. 4/5 P:861-932; readings R7-R10), the plain definition.
 * I/O i of device d (arrival a_i, completion c_i, both ns):
 *   q_now_i   = #{ j of d : (a_j, j) <= (a_i, i) and c_j > a_i }        (pending incl. self)
 *   C_i       = { j of d : c_j <= a_i }                                   (completed at issue)
 *   history   = the 4 largest members of C_i by (c_j, j); [0] = most recent
 *   lat_us[k] = floor((c_j - a_j) / 1000) (clamped to uint32), q_hist[k] = q_now_j; else 0.
 * dev may be NULL (one device). O(n^2): test sizes only. raw_out: uint32[n][9].
 */
void oracle_capture(const int64_t *a, const int64_t *c, const int32_t *dev, int64_t n,
                    uint32_t *raw_out)
{
    uint32_t *q = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(n > 0 ? n : 1));
    if (!q) return;
    for (int64_t i = 0; i < n; ++i) {
        uint32_t cnt = 0;
        for (int64_t j = 0; j < n; ++j) {
            if (dev && dev[j] != dev[i]) continue;
            int issued_before = (a[j] < a[i]) || (a[j] == a[i] && j <= i);
            if (issued_before && c[j] > a[i]) ++cnt;
        }
        q[i] = cnt;
    }
    for (int64_t i = 0; i < n; ++i) {
        int64_t top[4] = {-1, -1, -1, -1};   /* top[0] = largest (c_j, j) */
        for (int64_t j = 0; j < n; ++j) {
            if (dev && dev[j] != dev[i]) continue;
            if (c[j] > a[i]) continue;
            for (int k = 0; k < 4; ++k) {
                int64_t t = top[k];
                if (t < 0 || c[j] > c[t] || (c[j] == c[t] && j > t)) {
                    for (int m = 3; m > k; --m) top[m] = top[m - 1];
                    top[k] = j;
                    break;
                }
            }
        }
        uint32_t *r = raw_out + 9 * i;
        r[0] = q[i];
        for (int k = 0; k < 4; ++k) {
            if (top[k] >= 0) {
                int64_t us = (c[top[k]] - a[top[k]]) / 1000;
                r[1 + k] = us > 0xFFFFFFFFLL ? 0xFFFFFFFFu : (uint32_t)us;
                r[5 + k] = q[top[k]];
            } else {
                r[1 + k] = 0;
                r[5 + k] = 0;
            }
        }
    }
    free(q);
}

/* Same definition for selected rows only (O(n) per row): raw_out uint32[m][9] for rows[]. */
void oracle_capture_rows(const int64_t *a, const int64_t *c, const int32_t *dev, int64_t n,
                         const int64_t *rows, int64_t m, uint32_t *raw_out)
{
    for (int64_t r = 0; r < m; ++r) {
        const int64_t i = rows[r];
        uint32_t q = 0;
        int64_t top[4] = {-1, -1, -1, -1};
        for (int64_t j = 0; j < n; ++j) {
            if (dev && dev[j] != dev[i]) continue;
            int issued_before = (a[j] < a[i]) || (a[j] == a[i] && j <= i);
            if (issued_before && c[j] > a[i]) ++q;
            if (c[j] > a[i]) continue;
            for (int k = 0; k < 4; ++k) {
                int64_t t = top[k];
                if (t < 0 || c[j] > c[t] || (c[j] == c[t] && j > t)) {
                    for (int mm = 3; mm > k; --mm) top[mm] = top[mm - 1];
                    top[k] = j;
                    break;
                }
            }
        }
        uint32_t *o = raw_out + 9 * r;
        o[0] = q;
        for (int k = 0; k < 4; ++k) {
            if (top[k] >= 0) {
                const int64_t j = top[k];
                int64_t us = (c[j] - a[j]) / 1000;
                o[1 + k] = us > 0xFFFFFFFFLL ? 0xFFFFFFFFu : (uint32_t)us;
                uint32_t qj = 0;   /* q_now of j, by the same definition */
                for (int64_t jj = 0; jj < n; ++jj) {
                    if (dev && dev[jj] != dev[j]) continue;
                    int ib = (a[jj] < a[j]) || (a[jj] == a[j] && jj <= j);
                    if (ib && c[jj] > a[j]) ++qj;
                }
                o[5 + k] = qj;
            } else {
                o[1 + k] = 0;
                o[5 + k] = 0;
            }
        }
    }
}

/*
 * Second workload on the same fused-MLP family: the MLPs LAKE
 * ports for load balancing (MLLB, §7.3, Fig. 10) and readahead classification
 * (KML, §7.4, Fig. 11). PAPER.md gives no layer shapes or activations for
 * either; the shapes are readings (R25-R28) and this function takes them as
 * arguments. Plain definition, per input row i:
 *   h = x[i]
 *   for each hidden layer l: per output j, acc = +0.0f, acc = fmaf(h[k], W_l[j][k], acc)
 *       for k ascending, z = acc + b_l[j] (one rounding), then
 *       act 0 (ReLU):    h'[j] = (z > 0.0f) ? z : +0.0f          (R15, as for LinnOS)
 *       act 1 (sigmoid): h'[j] = 1.0f / (1.0f + expf(-z))        (R27)
 *   output layer (identity): out[c] = acc_c + b_out[c], c < C = widths[n_layers]
 *   class = the first c with out[c] maximal: best = 0; for c = 1..C-1, best = c when
 *           out[c] > out[best]  (R28; for C = 2 this is R14's decision; NaN never wins)
 * blob: per layer W_l[widths[l+1]][widths[l]] row-major then b_l[widths[l+1]].
 * x: float[n][widths[0]]; out: float[n][C] (may be NULL); cls: int32[n].
 */
int oracle_mlp_family(int n_layers, const int *widths, int act, const float *blob,
                      const float *x, int64_t n, float *out, int32_t *cls, int nthreads)
{
    if (n_layers < 1 || (act != 0 && act != 1) || widths[n_layers] < 2) return 1;
    int maxw = 0;
    for (int l = 0; l <= n_layers; ++l) {
        if (widths[l] <= 0) return 1;
        if (widths[l] > maxw) maxw = widths[l];
    }
    const int C = widths[n_layers];
#ifdef _OPENMP
    const int nt = nthreads > 0 ? nthreads : omp_get_num_procs();
#else
    (void)nthreads;
#endif
#pragma omp parallel for schedule(static) num_threads(nt)
    for (int64_t i = 0; i < n; ++i) {
        float bufa[maxw], bufb[maxw];
        float *h = bufa, *hn = bufb;
        memcpy(h, x + i * widths[0], sizeof(float) * (size_t)widths[0]);
        const float *p = blob;
        for (int l = 0; l < n_layers; ++l) {
            const int K = widths[l], N = widths[l + 1];
            const float *W = p;
            const float *b = p + (int64_t)N * K;
            p = b + N;
            const int hidden = (l + 1 < n_layers);
            for (int j = 0; j < N; ++j) {
                float acc = +0.0f;
                for (int k = 0; k < K; ++k) acc = fmaf(h[k], W[(int64_t)j * K + k], acc);
                float z = acc + b[j];
                if (!hidden) hn[j] = z;
                else if (act == 0) hn[j] = (z > 0.0f) ? z : 0.0f;
                else hn[j] = 1.0f / (1.0f + expf(-z));
            }
            float *t = h; h = hn; hn = t;
        }
        int best = 0;
        for (int c = 1; c < C; ++c)
            if (h[c] > h[best]) best = c;
        cls[i] = best;
        if (out) memcpy(out + i * C, h, sizeof(float) * (size_t)C);
    }
    return 0;
}

int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_num_procs();
#else
    return 1;
#endif
}
