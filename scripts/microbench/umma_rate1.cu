// Microbenchmark: cycles per tcgen05.mma.cta_group::1.kind::f16 (M = 128), A from TMEM or
// SMEM, B K-major or MN-major SWIZZLE_NONE, N = 64 / 128. One CTA, 4096 MMAs.
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_finglertyshar23_b200/csrc/lake_ptx.cuh"
using namespace lake;

__device__ __forceinline__ void mma1(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
               "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
               :: "r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
}
__device__ __forceinline__ void mma1_ts(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
               "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}"
               :: "r"(d), "r"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
}

template <int A_TMEM, int B_MN, int N>
__global__ void __launch_bounds__(128, 1) k(unsigned long long *out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sb = ptx::smem_u32(smem);
  const uint32_t warp = threadIdx.x >> 5;
  for (uint32_t i = threadIdx.x; i < 160 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = 0;
  const uint32_t bar = sb + 160 * 1024, slot = bar + 8;
  if (threadIdx.x == 0) { ptx::mbar_init(bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(slot), "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  ptx::fence_proxy_async_smem();
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + 160 * 1024 + 8);
  if (threadIdx.x == 0) {
    uint32_t idesc = ptx::umma_idesc_f16(0, 128, N) | (B_MN ? (1u << 16) : 0u);
    const uint64_t bdesc = ptx::umma_desc(sb + 65536, N * 16, 128);
    const uint32_t bstep = (2 * N * 16) >> 4;
    const uint64_t adesc = ptx::umma_desc(sb, 128 * 16, 128);
    const uint32_t d = tmem + 256;
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const uint32_t ks = i & 15;
      if (A_TMEM) mma1_ts(d, tmem + ks * 8, bdesc + ks * bstep, idesc, ks);
      else mma1(d, adesc + ks * ((2 * 128 * 16) >> 4), bdesc + ks * bstep, idesc, ks);
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(bar) : "memory");
    ptx::mbar_wait(bar, 0);
    out[0] = clock64() - t0;
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tmem), "r"(512));
  }
}

template <int A_TMEM, int B_MN, int N>
void run(const char *name) {
  unsigned long long *d, h = 0;
  cudaMalloc(&d, 8);
  auto f = k<A_TMEM, B_MN, N>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 170 * 1024);
  const int iters = 4096;
  for (int rep = 0; rep < 3; ++rep) {
    f<<<1, 128, 170 * 1024>>>(d, iters);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
  }
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  const double flop = 128.0 * N * 16 * 2;
  printf("%-28s %7.1f cycles/MMA  %6.0f FLOP/clk/SM (%.0f%% of 8192)\n", name, (double)h / iters,
         flop * iters / h, 100.0 * flop * iters / h / 8192);
  cudaFree(d);
}

int main() {
  run<1, 1, 64>("cg1 A=TMEM B=MN N=64");
  run<0, 1, 64>("cg1 A=SMEM B=MN N=64");
  run<0, 0, 64>("cg1 A=SMEM B=K  N=64");
  run<1, 1, 128>("cg1 A=TMEM B=MN N=128");
  run<0, 1, 128>("cg1 A=SMEM B=MN N=128");
  run<0, 0, 128>("cg1 A=SMEM B=K  N=128");
  return 0;
}
