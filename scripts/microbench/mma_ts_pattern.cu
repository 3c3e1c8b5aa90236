// Microbenchmark: the fused kernel's hidden-layer MMA pattern on one CTA pair.
// 16 x tcgen05.mma.cta_group::2.kind::f16 M=256 N=256 K=16 per "layer", A from TMEM at the
// kernel's column pattern (K-step s at column A_STRIDE*s), B K-major from SMEM, D in the
// other 256-column buffer; optional bias MMA (A from SMEM) first; optional per-chunk
// try_wait + fence + __syncwarp (warp-converged issue); optional 8 warps loading/storing the
// accumulator buffer's columns (tcgen05.ld x16 / st x8 + waits) like the epilogue.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o mma_ts_pattern mma_ts_pattern.cu
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_finglertyshar23_b200/csrc/lake_ptx.cuh"
using namespace lake;

template <int A_STRIDE, int BIAS, int EPI>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(320, 1) k(unsigned long long *out, int layers) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sb = ptx::smem_u32(smem);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ptx::cluster_ctarank();
  for (uint32_t i = threadIdx.x; i < 160 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = 0;
  const uint32_t bar = sb + 160 * 1024, slot = bar + 8, done = bar + 16, stop = bar + 24;
  if (threadIdx.x == 0) {
    ptx::mbar_init(bar, 1);
    ptx::mbar_init(done, 1);
    ptx::fence_mbar_init();
    *reinterpret_cast<volatile uint32_t *>(smem + 160 * 1024 + 24) = 0;
  }
  if (warp == 0) { ptx::tmem_alloc_cg2(slot, 512); ptx::tmem_relinquish_cg2(); }
  ptx::fence_proxy_async_smem();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  if (threadIdx.x == 0) ptx::mbar_arrive(bar);
  __syncthreads();
  const uint32_t tmem0 = *reinterpret_cast<volatile uint32_t *>(smem + 160 * 1024 + 8);
  volatile uint32_t *stopf = reinterpret_cast<volatile uint32_t *>(smem + 160 * 1024 + 24);
  if (warp == 0 && rank == 0) {
    const uint32_t tm = __shfl_sync(0xffffffffu, tmem0, 0);
    const bool issuer = lane == 0;
    const uint32_t idesc = ptx::umma_idesc_f16(0, 256, 256);
    const uint64_t bdesc = ptx::umma_desc(sb + 65536, 128 * 16, 128);
    const uint64_t adesc = ptx::umma_desc(sb, 128 * 16, 128);
    constexpr uint64_t kStep = (2 * 128 * 16) >> 4;
    unsigned long long t0 = clock64();
    for (int l = 0; l < layers; ++l) {
      const uint32_t d = tm + 256;  // D: columns 256-511, A: columns 0-255
      if (BIAS && issuer) ptx::mma_f16_cg2(d, adesc, bdesc, idesc, 0);
      for (uint32_t kc = 0; kc < 8; ++kc) {
        ptx::mbar_wait(bar, 0);
        ptx::tc_fence_after();
#pragma unroll
        for (uint32_t s = 0; s < 2; ++s) {
          const uint32_t ks = kc * 2 + s;
          if (issuer) ptx::mma_f16_cg2_ts(d, tm + A_STRIDE * ks, bdesc + ks * kStep, idesc, ks | BIAS);
        }
        __syncwarp();
      }
    }
    if (issuer) ptx::mma_commit_cg2(done, 0x3);
    ptx::mbar_wait(done, 0);
    unsigned long long t1 = clock64();
    if (issuer) { out[0] = t1 - t0; *stopf = 1; }
  } else if (EPI && rank == 0 && warp >= 2 && warp < 10) {
    // "epilogue": this warp's TMEM lane quadrant, columns 0-255 of the A buffer region
    // (as the kernel's epilogue works on the other buffer while the MMA runs)
    const uint32_t q = warp & 3;
    const uint32_t tb = tmem0 + ((q * 32) << 16);
    uint32_t r[16], p[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    uint32_t it = 0;
    while (!*stopf) {
      const uint32_t col = 128 + ((it * 16 + (warp >> 2) * 8) & 127);  // upper half of A buffer: untouched by the A reads
      ptx::tmem_ld_32x32b_x16(tb + col, r);
      ptx::tmem_ld_wait();
#pragma unroll
      for (int i = 0; i < 8; ++i) p[i] += r[2 * i] ^ r[2 * i + 1];
      ptx::tmem_st_32x32b_x8(tb + col, p);
      ptx::tmem_st_wait();
      ++it;
    }
  } else if (rank == 1 && threadIdx.x == 0) {
    ptx::mbar_wait(done, 0);
  }
  __syncwarp();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == 0) { ptx::tc_fence_after(); ptx::tmem_dealloc_cg2(tmem0, 512); }
}

template <int A_STRIDE, int BIAS, int EPI>
void run(const char *name) {
  unsigned long long *d, h = 0;
  cudaMalloc(&d, 8);
  auto f = k<A_STRIDE, BIAS, EPI>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 170 * 1024);
  const int layers = 256;
  for (int rep = 0; rep < 3; ++rep) {
    f<<<2, 320, 170 * 1024>>>(d, layers);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
  }
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("%-46s %7.1f cycles per layer (16 MMAs%s; ideal %d)\n", name, (double)h / layers,
         BIAS ? " + bias MMA" : "", BIAS ? 2176 : 2048);
  fflush(stdout);
  cudaFree(d);
}

int main() {
  run<8, 0, 0>("A cols 8s, no bias, no epilogue");
  run<16, 0, 0>("A cols 16s (kernel), no bias, no epilogue");
  run<16, 1, 0>("A cols 16s, bias MMA, no epilogue");
  run<16, 1, 1>("A cols 16s, bias MMA, 8 epilogue warps ld/st");
  run<8, 0, 1>("A cols 8s, no bias, 8 epilogue warps ld/st");
  return 0;
}
