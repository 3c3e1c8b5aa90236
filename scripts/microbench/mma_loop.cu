// Microbenchmark: cost of the MMA issuer's per-chunk loop in the fused kernels.
// One CTA pair; the leader's warp issues `chunks` K-chunks of 2 tcgen05.mma (cta_group::2,
// M=256 N=256 K=16, A and B from SMEM) and, per variant, a try_wait on an already-completed
// mbarrier, a tcgen05.commit per chunk, a __syncwarp. Prints cycles per chunk (ideal: 256).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o mma_loop mma_loop.cu
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_finglertyshar23_b200/csrc/lake_ptx.cuh"
using namespace lake;

template <int WAIT, int COMMIT, int WARP>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) k(unsigned long long *out, int chunks) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sb = ptx::smem_u32(smem);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ptx::cluster_ctarank();
  for (uint32_t i = threadIdx.x; i < 160 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = 0;
  const uint32_t bar = sb + 160 * 1024, slot = bar + 8, done = bar + 16, cbar = bar + 24;
  if (threadIdx.x == 0) {
    ptx::mbar_init(bar, 1);
    ptx::mbar_init(done, 1);
    for (int i = 0; i < 8; ++i) ptx::mbar_init(cbar + 8 * i, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 0) { ptx::tmem_alloc_cg2(slot, 512); ptx::tmem_relinquish_cg2(); }
  ptx::fence_proxy_async_smem();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  if (threadIdx.x == 0) ptx::mbar_arrive(bar);  // phase 0 of `bar` completes: waits pass at once
  __syncthreads();
  const uint32_t tmem0 = *reinterpret_cast<volatile uint32_t *>(smem + 160 * 1024 + 8);
  if (rank == 0 && warp == 0 && (WARP || lane == 0)) {
    const uint32_t tm = WARP ? __shfl_sync(0xffffffffu, tmem0, 0) : tmem0;
    const bool issuer = lane == 0;
    const uint32_t idesc = ptx::umma_idesc_f16(0, 256, 256);
    const uint64_t adesc = ptx::umma_desc(sb, 128 * 16, 128);
    const uint64_t bdesc = ptx::umma_desc(sb + 65536, 128 * 16, 128);
    constexpr uint64_t kStep = (2 * 128 * 16) >> 4;
    unsigned long long t0 = clock64();
    for (int c = 0; c < chunks; c += 8) {
#pragma unroll
      for (uint32_t kc = 0; kc < 8; ++kc) {
        if (WAIT) { ptx::mbar_wait(bar, 0); ptx::tc_fence_after(); }
#pragma unroll
        for (uint32_t s = 0; s < 2; ++s) {
          const uint32_t ks = kc * 2 + s;
          if (issuer) ptx::mma_f16_cg2(tm + 256 * (c & 8 ? 1 : 0), adesc + (kc * 8192 >> 4) + s * kStep,
                                       bdesc + ks * kStep, idesc, ks);
        }
        if (COMMIT && issuer) ptx::mma_commit_cg2(cbar + 8 * kc, 0x3);
        if (WARP) __syncwarp();
      }
    }
    if (issuer) ptx::mma_commit_cg2(done, 0x3);
    ptx::mbar_wait(done, 0);
    unsigned long long t1 = clock64();
    if (issuer) out[0] = t1 - t0;
  } else if (rank == 1 && threadIdx.x == 0) {
    ptx::mbar_wait(done, 0);
  }
  __syncwarp();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == 0) { ptx::tc_fence_after(); ptx::tmem_dealloc_cg2(tmem0, 512); }
}

template <int WAIT, int COMMIT, int WARP>
void run(const char *name) {
  unsigned long long *d, h = 0;
  cudaMalloc(&d, 8);
  auto f = k<WAIT, COMMIT, WARP>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 170 * 1024);
  const int chunks = 2048;
  for (int rep = 0; rep < 3; ++rep) {
    f<<<2, 128, 170 * 1024>>>(d, chunks);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
  }
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("%-44s %7.1f cycles/chunk (2 MMAs; ideal 256)\n", name, (double)h / chunks);
  cudaFree(d);
}

int main() {
  run<0, 0, 0>("lane0: MMAs only");
  run<1, 0, 0>("lane0: wait + MMAs");
  run<0, 1, 0>("lane0: MMAs + commit");
  run<1, 1, 0>("lane0: wait + MMAs + commit");
  run<0, 0, 1>("warp:  MMAs only");
  run<1, 0, 1>("warp:  wait + MMAs");
  run<0, 1, 1>("warp:  MMAs + commit");
  run<1, 1, 1>("warp:  wait + MMAs + commit");
  return 0;
}
