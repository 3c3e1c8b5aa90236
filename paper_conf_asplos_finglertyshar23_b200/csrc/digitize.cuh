// digitize.cuh — device-side digitisation of one raw I/O record (product path).
//
// Definition (BASELINE.json north_star; readings R1-R6 in DESIGN.md §3): the 31 LinnOS
// inputs are D3(q_now) | D4(lat_us[0..3]) | D3(q_hist[0..3]), where Dw(v) is the w
// decimal digits of min(v, 10^w - 1), most significant first. Feature semantics: PAPER.md
// §5.5, §7.1; history index 0 = most recent, §5.2 P:769-772.
//
// Integer only, so it is bit-exact by construction; the caller chooses what to do with the
// digits (bytes for lake_linnos_digitize, fp32 / fp16 / bf16 operands inside the fused
// kernels). Division by a constant compiles to multiply-high.
#pragma once
#include <cstdint>

#include "lake_internal.h"

namespace lake {

// Emit the w digits of min(v, 10^w-1) MSB-first through f(position, digit).
template <int W, typename F>
__device__ __forceinline__ void emit_digits(uint32_t v, int pos, F &&f) {
  constexpr uint32_t cap = (W == 3) ? 999u : 9999u;
  uint32_t m = v < cap ? v : cap;
  if constexpr (W == 4) {
    uint32_t d0 = m / 1000u;
    uint32_t r = m - d0 * 1000u;
    uint32_t d1 = r / 100u;
    r -= d1 * 100u;
    uint32_t d2 = r / 10u;
    uint32_t d3 = r - d2 * 10u;
    f(pos + 0, d0); f(pos + 1, d1); f(pos + 2, d2); f(pos + 3, d3);
  } else {
    uint32_t d0 = m / 100u;
    uint32_t r = m - d0 * 100u;
    uint32_t d1 = r / 10u;
    uint32_t d2 = r - d1 * 10u;
    f(pos + 0, d0); f(pos + 1, d1); f(pos + 2, d2);
  }
}

// rec = {q_now, lat_us[0..3], q_hist[0..3]}; f(position 0..30, digit 0..9).
template <typename F>
__device__ __forceinline__ void digitize_record(const uint32_t (&rec)[9], F &&f) {
  emit_digits<3>(rec[0], 0, f);
#pragma unroll
  for (int k = 0; k < 4; ++k) emit_digits<4>(rec[1 + k], 3 + 4 * k, f);
#pragma unroll
  for (int k = 0; k < 4; ++k) emit_digits<3>(rec[5 + k], 19 + 3 * k, f);
}

}  // namespace lake

namespace lake {

// Packed digit row (internal workspace format, 16 B per I/O): the digit of tensor-core slot s
// (tc_slot_digit, lake_internal.h) in nibble (s & 1) of byte s/2 (low nibble first); slot 31
// is 1 (the layer-0 bias input: W0's slot-31 column holds b0). Written by the grouping pass in model-grouped order so the fused tensor-core kernel
// can bulk-copy contiguous rows and turn each byte into one operand pair.
__device__ __forceinline__ uint4 pack_slots(const uint32_t (&dg)[32] /* canonical order */) {
  uint32_t w[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    uint32_t v = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j)
      v |= (q * 8 + j == 31 ? 1u : (dg[tc_slot_digit(q * 8 + j)] & 0xFu)) << (4 * j);
    w[q] = v;
  }
  return make_uint4(w[0], w[1], w[2], w[3]);
}

// Packed row of one raw record, reference form (digit by digit through pack_slots).
__device__ __forceinline__ uint4 pack_record_digits(const uint32_t (&rec)[9]) {
  uint32_t dg[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) dg[i] = 0;
  digitize_record(rec, [&](int k, uint32_t v) { dg[k] = v; });
  return pack_slots(dg);
}

// SWAR digit pairs: for two values a, b < 100 held as x = a | b << 16, returns
// p(a) | p(b) << 16 with p(y) = (y / 10) | (y % 10) << 4, the packed byte of a two-digit
// field (tens in slot 2p, ones in slot 2p+1). y / 10 = (y * 205) >> 11 for y < 1029; the
// halves cannot carry into each other (y * 205 < 2^15), and p(y) = 16 y - 159 (y / 10).
__host__ __device__ __forceinline__ uint32_t bcd_pair2(uint32_t x) {
  const uint32_t t = ((x * 205u) >> 11) & 0x000F000Fu;
  return 16u * x - 159u * t;
}
// Hundreds split of two values a, b <= 999 held as x = a | b << 16: hi = v / 100 per half
// ((v * 41) >> 12 for v <= 999: checked exhaustively by tests/test_pack_swar.py), lo = v - 100 hi.
__host__ __device__ __forceinline__ uint32_t hundreds_pair3(uint32_t x) {
  return ((x * 41u) >> 12) & 0x000F000Fu;
}

// Packed row of one raw record (same bytes as pack_record_digits; ~90 integer ops instead of
// ~230: the grouping pass that writes these rows was ALU-issue bound on the digit-by-digit
// form). Layout (tc_slot_digit): bytes 0-7 = p(lat_f / 100), p(lat_f % 100) for f = 0..3;
// bytes 8-12 = p(q % 100) for q_now, q_hist[0..3]; bytes 13-15 = the five leading queue
// digits paired low-nibble first, then the constant 1 of slot 31.
__host__ __device__ __forceinline__ uint4 pack_record(const uint32_t (&rec)[9]) {
  uint32_t w01[2];
#pragma unroll
  for (int k = 0; k < 2; ++k) {  // two latency fields per word
    uint32_t half[2];
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      const uint32_t v = rec[1 + 2 * k + j] < 9999u ? rec[1 + 2 * k + j] : 9999u;
      const uint32_t hi = (v * 5243u) >> 19;  // v / 100 for v < 43699
      const uint32_t p = bcd_pair2(hi | (v - 100u * hi) << 16);
      half[j] = (p & 0xFFu) | ((p >> 8) & 0xFF00u);
    }
    w01[k] = half[0] | half[1] << 16;
  }
  uint32_t q[5];
#pragma unroll
  for (int g = 0; g < 5; ++g) {
    const uint32_t r = g == 0 ? rec[0] : rec[4 + g];
    q[g] = r < 999u ? r : 999u;
  }
  const uint32_t x01 = q[0] | q[1] << 16, x23 = q[2] | q[3] << 16;
  const uint32_t h01 = hundreds_pair3(x01), h23 = hundreds_pair3(x23), h4 = (q[4] * 41u) >> 12;
  const uint32_t p01 = bcd_pair2(x01 - 100u * h01), p23 = bcd_pair2(x23 - 100u * h23);
  const uint32_t p4 = bcd_pair2(q[4] - 100u * h4);
  const uint32_t w2 = (p01 & 0xFFu) | ((p01 >> 8) & 0xFF00u) | (p23 & 0xFFu) << 16 |
                      ((p23 >> 16) & 0xFFu) << 24;
  const uint32_t w3 = (p4 & 0xFFu) | (h01 & 0xFu) << 8 | (h01 >> 16) << 12 | (h23 & 0xFu) << 16 |
                      (h23 >> 16) << 20 | h4 << 24 | 1u << 28;
  return make_uint4(w01[0], w01[1], w2, w3);
}

// Packed row of a LAKE_IN_DIGITS row (bytes 0..30 are digits 0..9).
__device__ __forceinline__ uint4 pack_digit_bytes(const uint4 lo, const uint4 hi) {
  const uint32_t b[8] = {lo.x, lo.y, lo.z, lo.w, hi.x, hi.y, hi.z, hi.w};
  uint32_t dg[32];
#pragma unroll
  for (int k = 0; k < 32; ++k) dg[k] = k < 31 ? (b[k >> 2] >> ((k & 3) * 8)) & 0xFFu : 0u;
  return pack_slots(dg);
}

}  // namespace lake
