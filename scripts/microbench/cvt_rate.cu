// Microbenchmark: per-SM throughput of the epilogue's ALU ops (results per clock per SM):
// F2FP (cvt.rn.relu.f16x2.f32: 2 fp32 -> packed fp16 pair), FADD, HFMA2.RELU, FMNMX.
#include <cstdio>
#include <cstdint>

template <int OP>
__global__ void k(uint32_t *out, unsigned long long *cyc, int iters) {
  float a[16];
  uint32_t u[16];
  for (int i = 0; i < 16; ++i) { a[i] = threadIdx.x * 0.001f + i; u[i] = threadIdx.x + i; }
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      if (OP == 0) asm volatile("cvt.rn.relu.f16x2.f32 %0, %1, %2;" : "=r"(u[i]) : "f"(a[i]), "f"(a[(i + 1) & 15]));
      if (OP == 1) asm volatile("add.f32 %0, %0, %1;" : "+f"(a[i]) : "f"(a[(i + 3) & 15]));
      if (OP == 2) asm volatile("fma.rn.relu.f16x2 %0, %0, %1, %2;" : "+r"(u[i]) : "r"(u[(i + 1) & 15]), "r"(u[(i + 2) & 15]));
      if (OP == 3) asm volatile("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(u[i]) : "f"(a[i]), "f"(a[(i + 1) & 15]));
      if (OP == 4) asm volatile("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(u[i]) : "f"(a[i]), "f"(a[(i + 1) & 15]));
      if (OP == 0 || OP == 3 || OP == 4) a[i] = __uint_as_float(u[i] ^ 0x1000);  // keep a dependency-free stream
    }
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  uint32_t s = 0;
  for (int i = 0; i < 16; ++i) s ^= u[i] ^ __float_as_uint(a[i]);
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int OP>
void run(const char *name, int threads) {
  uint32_t *o; unsigned long long *c, h;
  cudaMalloc(&o, 1 << 20); cudaMalloc(&c, 8 * 148);
  const int iters = 2000;
  k<OP><<<148, threads>>>(o, c, iters);
  k<OP><<<148, threads>>>(o, c, iters);
  cudaDeviceSynchronize();
  cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
  const double ops = (double)threads * iters * 16;  // thread-instructions per SM
  printf("%-34s %4d thr: %6.1f thread-instr/clk/SM\n", name, threads, ops / h);
  cudaFree(o); cudaFree(c);
}

int main() {
  for (int t : {256, 512, 1024}) {
    run<0>("cvt.rn.relu.f16x2.f32 (F2FP)", t);
    run<3>("cvt.rn.f16x2.f32", t);
    run<4>("cvt.rn.bf16x2.f32", t);
    run<1>("add.f32", t);
    run<2>("fma.rn.relu.f16x2", t);
  }
  return 0;
}
