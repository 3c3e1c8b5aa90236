// Microbenchmark: cycles per tcgen05.mma.cta_group::2.kind::f16 for the operand
// configurations the fused kernel can use (A from TMEM or SMEM, B K-major or MN-major
// SWIZZLE_NONE, N = 16 .. 256). One CTA pair, one issuing thread, 4096 MMAs back to back.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o umma_rate umma_rate.cu
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_finglertyshar23_b200/csrc/lake_ptx.cuh"
using namespace lake;

template <int A_TMEM, int B_MN, int N, int SBO_PAD>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) k(unsigned long long *out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sb = ptx::smem_u32(smem);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
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
    uint32_t idesc = ptx::umma_idesc_f16(0, 256, N) | (B_MN ? (1u << 16) : 0u);
    // B: N/2 rows per CTA, K = 256
    const uint32_t nh = N / 2;
    uint64_t bdesc;
    uint32_t bstep;
    if (B_MN) {  // (k-group) stride LBO = nh*16 (n-groups adjacent), n-group stride SBO = 128
      bdesc = ptx::umma_desc(sb + 65536, nh * 16, 128 + SBO_PAD);
      bstep = (2 * nh * 16) >> 4;
    } else {     // K-major: core (rg, kg) at kg*(nh*16) + rg*128
      bdesc = ptx::umma_desc(sb + 65536, nh * 16, 128);
      bstep = (2 * nh * 16) >> 4;
    }
    const uint64_t adesc = ptx::umma_desc(sb, 128 * 16, 128);
    const uint32_t d = tmem + 256;
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const uint32_t ks = i & 15;
      if (A_TMEM) ptx::mma_f16_cg2_ts(d, tmem + ks * 8, bdesc + ks * bstep, idesc, ks);
      else ptx::mma_f16_cg2(d, adesc + ks * ((2 * 128 * 16) >> 4), bdesc + ks * bstep, idesc, ks);
    }
    ptx::mma_commit_cg2(bar, 0x3);
    ptx::mbar_wait(bar, 0);
    unsigned long long t1 = clock64();
    out[0] = t1 - t0;
  } else if (rank == 1 && threadIdx.x == 0) {
    ptx::mbar_wait(bar, 0);
  }
  __syncwarp();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == 0) { ptx::tc_fence_after(); ptx::tmem_dealloc_cg2(tmem, 512); }
}

template <int A_TMEM, int B_MN, int N, int SBO_PAD>
void run(const char *name) {
  unsigned long long *d, h = 0;
  cudaMalloc(&d, 8);
  auto f = k<A_TMEM, B_MN, N, SBO_PAD>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 170 * 1024);
  const int iters = 4096;
  for (int rep = 0; rep < 3; ++rep) {
    f<<<2, 128, 170 * 1024>>>(d, iters);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
  }
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  const double flop_per_sm = 128.0 * N * 16 * 2;  // per instruction per SM
  printf("%-34s %7.1f cycles/MMA  %6.0f FLOP/clk/SM (%.0f%% of 8192)\n", name, (double)h / iters,
         flop_per_sm * iters / h, 100.0 * flop_per_sm * iters / h / 8192);
  cudaFree(d);
}

int main() {
  run<1, 1, 128, 0>("A=TMEM B=MN  N=128");
  run<1, 0, 128, 0>("A=TMEM B=K   N=128");
  run<0, 1, 128, 0>("A=SMEM B=MN  N=128");
  run<0, 0, 128, 0>("A=SMEM B=K   N=128");
  run<1, 1, 256, 0>("A=TMEM B=MN  N=256");
  run<1, 0, 256, 0>("A=TMEM B=K   N=256");
  run<0, 0, 256, 0>("A=SMEM B=K   N=256");
  run<1, 1, 128, 16>("A=TMEM B=MN  N=128 sbo+16");
  // the NN output layer (N = 16) and neighbours
  run<1, 0, 16, 0>("A=TMEM B=K   N=16");
  run<0, 0, 16, 0>("A=SMEM B=K   N=16");
  run<1, 0, 32, 0>("A=TMEM B=K   N=32");
  run<1, 0, 64, 0>("A=TMEM B=K   N=64");
  return 0;
}
