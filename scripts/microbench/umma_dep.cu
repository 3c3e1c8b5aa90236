// Microbenchmark: is the >= 64-cycle cost of a narrow (N = 16) tcgen05.mma.cta_group::2
// (M = 256) a dependency on the accumulator it updates, or a per-instruction floor?
// The MMAs rotate over ND distinct accumulators (each a 16-column TMEM block); A from TMEM
// (the NN output layer's operand), B K-major SWIZZLE_NONE. One CTA pair, one issuing thread.
// Also: interleaving N = 16 MMAs with N = 256 MMAs (layer 0 of the next tile running
// between the output layer's K-steps).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o umma_dep umma_dep.cu
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_finglertyshar23_b200/csrc/lake_ptx.cuh"
using namespace lake;

// MIX = 0: all MMAs N; MIX = k > 0: after every k narrow MMAs, one N = 256 MMA to a separate
// accumulator (cycles reported per narrow MMA, net of nothing: the total is printed too).
template <int N, int ND, int MIX>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) k(unsigned long long *out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sb = ptx::smem_u32(smem);
  const uint32_t warp = threadIdx.x >> 5;
  const uint32_t rank = ptx::cluster_ctarank();
  for (uint32_t i = threadIdx.x; i < 160 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = 0;
  const uint32_t bar = sb + 160 * 1024, slot = bar + 8;
  if (threadIdx.x == 0) { ptx::mbar_init(bar, 1); ptx::fence_mbar_init(); }
  if (warp == 0) { ptx::tmem_alloc_cg2(slot, 512); ptx::tmem_relinquish_cg2(); }
  ptx::fence_proxy_async_smem();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + 160 * 1024 + 8);
  if (rank == 0 && threadIdx.x == 0) {
    const uint32_t idesc = ptx::umma_idesc_f16(0, 256, N);
    const uint32_t idesc_w = ptx::umma_idesc_f16(0, 256, 256);
    const uint32_t nh = N / 2;
    const uint64_t bdesc = ptx::umma_desc(sb + 65536, nh * 16, 128);
    const uint32_t bstep = (2 * nh * 16) >> 4;
    const uint64_t bdesc_w = ptx::umma_desc(sb + 65536, 128 * 16, 128);
    const uint32_t bstep_w = (2 * 128 * 16) >> 4;
    unsigned long long t0 = clock64();
    int wide = 0;
    for (int i = 0; i < iters; ++i) {
      const uint32_t ks = i & 15;
      const uint32_t d = tmem + 256 + (uint32_t)(i % ND) * 16;
      ptx::mma_f16_cg2_ts(d, tmem + ks * 8, bdesc + ks * bstep, idesc, (uint32_t)(i >= ND));
      if (MIX > 0 && (i % MIX) == MIX - 1) {
        // wide MMA into columns [0, 256) would overlap A (cols 0..127): use A cols 128..255
        // as both; the benchmark only measures timing, values are irrelevant.
        ptx::mma_f16_cg2_ts(tmem + 0, tmem + 128 + (wide & 7) * 8, bdesc_w + (wide & 7) * bstep_w, idesc_w, wide > 0);
        ++wide;
      }
    }
    ptx::mma_commit_cg2(bar, 0x3);
    ptx::mbar_wait(bar, 0);
    unsigned long long t1 = clock64();
    out[0] = t1 - t0;
    out[1] = (unsigned long long)wide;
  } else if (rank == 1 && threadIdx.x == 0) {
    ptx::mbar_wait(bar, 0);
  }
  __syncwarp();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == 0) { ptx::tc_fence_after(); ptx::tmem_dealloc_cg2(tmem, 512); }
}

template <int N, int ND, int MIX>
void run(const char *name) {
  unsigned long long *d, h[2] = {0, 0};
  cudaMalloc(&d, 16);
  auto f = k<N, ND, MIX>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 170 * 1024);
  const int iters = 4096;
  for (int rep = 0; rep < 3; ++rep) {
    f<<<2, 128, 170 * 1024>>>(d, iters);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
  }
  cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
  printf("%-40s total %9llu cycles  %7.1f cycles per narrow MMA  (%llu wide MMAs = %.0f cycles nominal)\n",
         name, h[0], (double)h[0] / iters, h[1], 128.0 * h[1]);
  cudaFree(d);
}

int main() {
  run<16, 1, 0>("N=16 one accumulator");
  run<16, 2, 0>("N=16 two accumulators");
  run<16, 4, 0>("N=16 four accumulators");
  run<16, 8, 0>("N=16 eight accumulators");
  run<32, 1, 0>("N=32 one accumulator");
  run<32, 4, 0>("N=32 four accumulators");
  run<64, 1, 0>("N=64 one accumulator");
  run<64, 4, 0>("N=64 four accumulators");
  run<16, 1, 16>("N=16 x16 + one N=256 per 16");
  run<16, 1, 8>("N=16 x8 + one N=256 per 8");
  run<16, 1, 2>("N=16 x2 + one N=256 per 2");
  run<16, 4, 4>("N=16 (4 acc) x4 + one N=256 per 4");
  return 0;
}
