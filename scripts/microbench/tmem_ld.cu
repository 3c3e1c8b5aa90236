// Microbenchmark: TMEM -> register load throughput on sm_100a (tcgen05.ld 32x32b).
// One CTA per SM, NW warps (multiple of 4); each warp loads its lane quadrant, x32 columns
// per instruction, ITER times, with a wait after every DEPTH loads. Reports bytes/clk/SM.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int DEPTH>
__global__ void __launch_bounds__(512, 1) k(int iters, unsigned long long *out, uint32_t *sink) {
  __shared__ uint32_t taddr_s;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&taddr_s)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tbase = taddr_s + (((warp & 3) * 32) << 16);
  uint32_t acc = 0;
  __syncthreads();
  const unsigned long long t0 = clock64();
  for (int i = 0; i < iters; i += DEPTH) {
    uint32_t r[DEPTH][32];
#pragma unroll
    for (int d = 0; d < DEPTH; ++d) {
      const uint32_t col = ((i + d) * 32 + (warp >> 2) * 64) & 511;
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
          : "=r"(r[d][0]), "=r"(r[d][1]), "=r"(r[d][2]), "=r"(r[d][3]), "=r"(r[d][4]), "=r"(r[d][5]), "=r"(r[d][6]), "=r"(r[d][7]), "=r"(r[d][8]), "=r"(r[d][9]), "=r"(r[d][10]), "=r"(r[d][11]), "=r"(r[d][12]), "=r"(r[d][13]), "=r"(r[d][14]), "=r"(r[d][15]), "=r"(r[d][16]), "=r"(r[d][17]), "=r"(r[d][18]), "=r"(r[d][19]), "=r"(r[d][20]), "=r"(r[d][21]), "=r"(r[d][22]), "=r"(r[d][23]), "=r"(r[d][24]), "=r"(r[d][25]), "=r"(r[d][26]), "=r"(r[d][27]), "=r"(r[d][28]), "=r"(r[d][29]), "=r"(r[d][30]), "=r"(r[d][31])
          : "r"(tbase + col));
    }
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int d = 0; d < DEPTH; ++d)
#pragma unroll
      for (int j = 0; j < 32; ++j) acc += r[d][j];
  }
  const unsigned long long t1 = clock64();
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
  sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(taddr_s));
}

template <int DEPTH>
void run(int nw, int iters) {
  const int blocks = 148;
  unsigned long long *out;
  uint32_t *sink;
  cudaMalloc(&out, blocks * 8);
  cudaMalloc(&sink, blocks * 512 * 4);
  k<DEPTH><<<blocks, nw * 32>>>(iters, out, sink);
  k<DEPTH><<<blocks, nw * 32>>>(iters, out, sink);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long h[148];
  cudaMemcpy(h, out, blocks * 8, cudaMemcpyDeviceToHost);
  unsigned long long mx = 0;
  for (int i = 0; i < blocks; ++i) mx = h[i] > mx ? h[i] : mx;
  const double bytes = (double)nw * iters * 32 * 32 * 4;
  printf("warps %2d depth %d: %s %llu cycles, %.1f B/clk/SM, %.1f cycles per warp-ld\n", nw, DEPTH,
         cudaGetErrorString(e), mx, bytes / mx, (double)mx / iters);
  cudaFree(out);
  cudaFree(sink);
}

int main() {
  for (int nw : {4, 8, 16}) {
    run<1>(nw, 4096);
    run<2>(nw, 4096);
    run<4>(nw, 4096);
  }
  return 0;
}
