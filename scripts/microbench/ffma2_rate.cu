// Microbenchmark: FP32 FMA throughput per SM, scalar FFMA vs packed FFMA2 (fma.rn.f32x2),
// 148 x k CTAs of 256 threads, 8 independent accumulator chains per thread.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ffma2_rate ffma2_rate.cu
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ unsigned long long f2(float a, float b) {
  unsigned long long r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
template <int PACKED>
__global__ void k(float *out, int iters, float s) {
  if (PACKED) {
    unsigned long long acc[8], x = f2(s, s + 1.0f), y = f2(1.0001f, 0.9999f);
    for (int i = 0; i < 8; ++i) acc[i] = f2((float)i, (float)(i + threadIdx.x));
    for (int it = 0; it < iters; ++it)
#pragma unroll
      for (int i = 0; i < 8; ++i)
        asm volatile("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc[i]) : "l"(x), "l"(y));
    float t = 0;
    for (int i = 0; i < 8; ++i) { float a, b; asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(acc[i])); t += a + b; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
  } else {
    float acc[16];
    for (int i = 0; i < 16; ++i) acc[i] = (float)(i + threadIdx.x);
    for (int it = 0; it < iters; ++it)
#pragma unroll
      for (int i = 0; i < 16; ++i) asm volatile("fma.rn.f32 %0, %1, %2, %0;" : "+f"(acc[i]) : "f"(s), "f"(1.0001f));
    float t = 0;
    for (int i = 0; i < 16; ++i) t += acc[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
  }
}
int main() {
  float *d; cudaMalloc(&d, 148 * 8 * 256 * 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  for (int packed = 0; packed < 2; ++packed)
    for (int blocks = 2; blocks <= 8; blocks *= 2) {
      const int iters = 20000;
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(a);
        if (packed) k<1><<<sms * blocks, 256>>>(d, iters, 0.5f); else k<0><<<sms * blocks, 256>>>(d, iters, 0.5f);
        cudaEventRecord(b); cudaEventSynchronize(b);
      }
      float ms; cudaEventElapsedTime(&ms, a, b);
      const double fmas = (double)sms * blocks * 256 * iters * 16;  // 16 FMAs per thread-iteration either way
      printf("%s blocks/SM %d: %.1f TFLOP/s, %.0f FMA/clk/SM at %.0f MHz (nominal clock)\n", packed ? "FFMA2" : "FFMA ",
             blocks, 2 * fmas / ms / 1e9, fmas / (ms * 1e-3) / sms / (clk * 1e3), clk / 1e3);
    }
  return 0;
}
