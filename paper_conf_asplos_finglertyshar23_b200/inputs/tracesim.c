/*
 * tracesim.c — deterministic event simulation behind the seeded synthetic I/O traces.
 *
 * Part of the seeded INPUT GENERATOR (paper_conf_asplos_finglertyshar23_b200/inputs/),
 * which serves both the oracle tests and the CUDA path. It holds none of the method's
 * arithmetic (no digitisation, no MLP): it only turns a trace (arrival time and service
 * demand per I/O, all random draws made by numpy PCG64 and passed in) into the raw
 * feature records the LinnOS registry would have captured (Fig. 4/5):
 *
 *   q_now     pending I/Os on the device at issue, INCLUDING the arriving I/O
 *             (Fig. 4 line 8 increments pend_ios before commit; reading R9)
 *   lat_us[k] latency of the k-th most recently completed I/O, k = 0 most recent
 *             (schema history idiom; LinnOS semantics, reading R10)
 *   q_hist[k] that completed I/O's own q_now at its issue
 *
 * Device model (the paper used real NVMe; entirely silent): an M/G/c FIFO
 * server with c channels. A completion at exactly the arrival instant counts as completed;
 * completion order is (complete_ns, index) ascending. Missing history is zero (R7).
 */
#include <stdint.h>
#include <stdlib.h>

typedef struct { int64_t t; int64_t i; } ev_t;

static int ev_less(ev_t a, ev_t b) { return a.t < b.t || (a.t == b.t && a.i < b.i); }

static void heap_push(ev_t *h, int64_t *sz, ev_t e)
{
    int64_t k = (*sz)++;
    h[k] = e;
    while (k > 0) {
        int64_t p = (k - 1) / 2;
        if (!ev_less(h[k], h[p])) break;
        ev_t t = h[k]; h[k] = h[p]; h[p] = t;
        k = p;
    }
}

static ev_t heap_pop(ev_t *h, int64_t *sz)
{
    ev_t top = h[0];
    h[0] = h[--(*sz)];
    int64_t k = 0;
    for (;;) {
        int64_t l = 2 * k + 1, r = l + 1, m = k;
        if (l < *sz && ev_less(h[l], h[m])) m = l;
        if (r < *sz && ev_less(h[r], h[m])) m = r;
        if (m == k) break;
        ev_t t = h[k]; h[k] = h[m]; h[m] = t;
        k = m;
    }
    return top;
}

/*
 * arrival_ns[n] non-decreasing; service_ns[n] > 0; channels >= 1.
 * Outputs: complete_ns[n]; raw[n][9] = {q_now, lat_us[0..3], q_hist[0..3]}.
 * Returns 0, or -1 on allocation failure / bad arguments.
 */
int tracesim_run(const int64_t *arrival_ns, const int64_t *service_ns, int64_t n, int channels,
                 int64_t *complete_ns, uint32_t *raw)
{
    if (n < 0 || channels < 1) return -1;
    if (n == 0) return 0;
    int64_t *chan_free = (int64_t *)calloc((size_t)channels, sizeof(int64_t));
    ev_t *heap = (ev_t *)malloc(sizeof(ev_t) * (size_t)n);
    uint32_t *qnow = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)n);
    if (!chan_free || !heap || !qnow) {
        free(chan_free); free(heap); free(qnow);
        return -1;
    }
    /* FIFO c-server: I/O i starts on the earliest-free channel at max(arrival, free). */
    for (int64_t i = 0; i < n; ++i) {
        int best = 0;
        for (int c = 1; c < channels; ++c)
            if (chan_free[c] < chan_free[best]) best = c;
        int64_t start = arrival_ns[i] > chan_free[best] ? arrival_ns[i] : chan_free[best];
        complete_ns[i] = start + service_ns[i];
        chan_free[best] = complete_ns[i];
    }
    /* Feature capture in arrival order. */
    int64_t hsz = 0;
    int64_t hist[4] = {-1, -1, -1, -1}; /* hist[0] = most recent completed I/O index */
    for (int64_t i = 0; i < n; ++i) {
        while (hsz > 0 && heap[0].t <= arrival_ns[i]) {
            ev_t e = heap_pop(heap, &hsz);
            hist[3] = hist[2]; hist[2] = hist[1]; hist[1] = hist[0]; hist[0] = e.i;
        }
        qnow[i] = (uint32_t)(hsz + 1);
        uint32_t *r = raw + 9 * i;
        r[0] = qnow[i];
        for (int k = 0; k < 4; ++k) {
            if (hist[k] >= 0) {
                int64_t j = hist[k];
                int64_t lat_ns = complete_ns[j] - arrival_ns[j];
                int64_t us = lat_ns / 1000;                 /* floor(ns/1000), R8 */
                r[1 + k] = us > 0xFFFFFFFFLL ? 0xFFFFFFFFu : (uint32_t)us;
                r[5 + k] = qnow[j];
            } else {
                r[1 + k] = 0;
                r[5 + k] = 0;
            }
        }
        ev_t e = {complete_ns[i], i};
        heap_push(heap, &hsz, e);
    }
    free(chan_free); free(heap); free(qnow);
    return 0;
}

/* Two-state "GC" Markov modulator: state[i] in {0,1}; enter with p_enter, leave with
 * p_leave per I/O; u[n] are U(0,1) draws made by the caller. */
void tracesim_markov(const double *u, int64_t n, double p_enter, double p_leave, uint8_t *state)
{
    int s = 0;
    for (int64_t i = 0; i < n; ++i) {
        if (s == 0) s = (u[i] < p_enter) ? 1 : 0;
        else        s = (u[i] < p_leave) ? 0 : 1;
        state[i] = (uint8_t)s;
    }
}
