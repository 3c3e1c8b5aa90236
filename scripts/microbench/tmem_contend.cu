// Microbenchmark: tcgen05.ld (32x32b.x32) latency and TMEM->RF bandwidth with and without
// concurrent tcgen05.mma traffic (cta_group::2, M=256, N=128, A from TMEM, B from SMEM), and
// the MMA rate itself while the load warps run (ST=1: each load is followed by a 16-column
// tcgen05.st, the H write-back of the fused kernel).
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_finglertyshar23_b200/csrc/lake_ptx.cuh"
using namespace lake;

template <int WITH_MMA, int NLD_WARPS, int ST = 0>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(32 * (NLD_WARPS + 1), 1)
k(unsigned long long *out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sb = ptx::smem_u32(smem);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ptx::cluster_ctarank();
  for (uint32_t i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = 0;
  const uint32_t bar = sb + 64 * 1024, slot = bar + 8, flag = bar + 16;
  if (threadIdx.x == 0) { ptx::mbar_init(bar, 1); ptx::fence_mbar_init(); *reinterpret_cast<volatile uint32_t *>(smem + 64 * 1024 + 16) = 0; }
  if (warp == 0) { ptx::tmem_alloc_cg2(slot, 512); ptx::tmem_relinquish_cg2(); }
  ptx::fence_proxy_async_smem();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + 64 * 1024 + 8);
  volatile uint32_t *stop = reinterpret_cast<volatile uint32_t *>(smem + 64 * 1024 + 16);
  if (warp == NLD_WARPS) {
    if (WITH_MMA && rank == 0 && lane == 0) {
      const uint32_t idesc = ptx::umma_idesc_f16(0, 256, 128) | (1u << 16);
      const uint64_t bdesc = ptx::umma_desc(sb, 1024, 128);
      const unsigned long long m0 = clock64();
      for (int i = 0; i < 16 * iters; ++i) {
        const uint32_t ks = i & 15;
        ptx::mma_f16_cg2_ts(tmem + 256 + ((i >> 4) & 1) * 128, tmem + ks * 8, bdesc + ks * 128, idesc, ks);
      }
      ptx::mma_commit_cg2(bar, 0x3);
      ptx::mbar_wait(bar, 0);
      out[126] = (clock64() - m0);
      out[127] = 16ull * iters;
    }
  } else {
    // loads from columns the MMA does not write (the A region 0..255)
    const uint32_t q = warp & 3;
    const uint32_t ta = tmem + ((q * 32) << 16) + (warp >> 2) * 32;
    uint32_t acc = 0;
    unsigned long long lat = 0;
    const unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      uint32_t r[32];
      const unsigned long long a = clock64();
      ptx::tmem_ld_32x32b_x32(ta + (i & 3) * 64, r);
      ptx::tmem_ld_wait();
      if (ST) {
        uint32_t w[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) w[j] = r[j] ^ r[j + 16];
        ptx::tmem_st_32x32b_x16(ta + (i & 3) * 64 + 128, w);
        ptx::tmem_st_wait();
      }
#pragma unroll
      for (int j = 0; j < 32; ++j) acc += r[j];
      lat += clock64() - a;
    }
    const unsigned long long t1 = clock64();
    if (lane == 0 && rank == 0) {
      out[warp * 2] = lat / iters;
      out[warp * 2 + 1] = t1 - t0;
    }
    if (acc == 0xdeadbeef) out[100] = acc;
  }
  if (WITH_MMA && threadIdx.x == 0 && rank == 1) ptx::mbar_wait(bar, 0);
  __syncwarp();
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == 0) { ptx::tc_fence_after(); ptx::tmem_dealloc_cg2(tmem, 512); }
}

template <int WITH_MMA, int NW, int ST = 0>
void run(const char *name) {
  unsigned long long *d, h[64] = {};
  cudaMalloc(&d, 8 * 128);
  cudaMemset(d, 0, 8 * 128);
  auto f = k<WITH_MMA, NW, ST>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 70 * 1024);
  const int iters = 2000;
  for (int rep = 0; rep < 2; ++rep) {
    f<<<2, 32 * (NW + 1), 70 * 1024>>>(d, iters);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
  }
  unsigned long long hm[2] = {};
  cudaMemcpy(h, d, 8 * 64, cudaMemcpyDeviceToHost);
  cudaMemcpy(hm, d + 126, 16, cudaMemcpyDeviceToHost);
  double bw = 0;
  unsigned long long lat = 0;
  for (int w = 0; w < NW; ++w) { lat += h[w * 2]; bw += 4096.0 * iters / h[w * 2 + 1]; }
  printf("%-24s %2d ld warps: ld x32 latency %5llu cycles, TMEM->RF %6.0f B/clk/SM", name, NW, NW ? lat / (NW ? NW : 1) : 0ull, bw);
  if (WITH_MMA) printf(", MMA %.1f cycles each (64 = full rate)", (double)hm[0] / hm[1]);
  printf("\n");
  cudaFree(d);
}

int main() {
  run<0, 4>("no MMA");
  run<1, 4>("with MMA");
  run<0, 8>("no MMA");
  run<1, 8>("with MMA");
  run<0, 16>("no MMA");
  run<1, 16>("with MMA");
  run<1, 0>("MMA alone");
  run<1, 8, 1>("with MMA, ld+st");
  run<1, 16, 1>("with MMA, ld+st");
  return 0;
}
