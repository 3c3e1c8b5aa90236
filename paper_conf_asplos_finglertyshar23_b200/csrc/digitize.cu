// digitize.cu — standalone digitisation kernel (lake_linnos_digitize): 36 B raw record in,
// 32 B digit row out, integer only (bit-exact). HBM-bound: 68 algorithmic bytes per I/O.
//
// A block stages 256 records (9216 B) into shared memory with coalesced 16-byte loads
// (4-byte loads for a misaligned base or a partial block), then each thread digitises one
// record (stride-9 word reads from SMEM are bank-conflict free) and writes its 32 output
// bytes as two 16-byte stores (consecutive threads -> consecutive 32 B).
#include "digitize.cuh"
#include "lake_internal.h"

namespace lake {
namespace {

constexpr int kDigBlock = 256;

__global__ void __launch_bounds__(kDigBlock)
digitize_kernel(const uint32_t *__restrict__ raw, int64_t n, uint8_t *__restrict__ out,
                bool vec_in, bool vec_out) {
  __shared__ __align__(16) uint32_t stage[kDigBlock * 9];
  const int tid = threadIdx.x;
  const int64_t nblocks = (n + kDigBlock - 1) / kDigBlock;
  for (int64_t blk = blockIdx.x; blk < nblocks; blk += gridDim.x) {
    const int64_t base = blk * kDigBlock;
    const int cnt = (int)((n - base) < kDigBlock ? (n - base) : kDigBlock);
    const uint32_t *src = raw + base * 9;
    if (vec_in && cnt == kDigBlock) {
      const uint4 *s4 = reinterpret_cast<const uint4 *>(src);
      uint4 *d4 = reinterpret_cast<uint4 *>(stage);
#pragma unroll
      for (int i = tid; i < kDigBlock * 9 / 4; i += kDigBlock) d4[i] = __ldcs(s4 + i);
    } else {
      for (int i = tid; i < cnt * 9; i += kDigBlock) stage[i] = __ldcs(src + i);
    }
    __syncthreads();
    if (tid < cnt) {
      uint32_t rec[9];
#pragma unroll
      for (int f = 0; f < 9; ++f) rec[f] = stage[tid * 9 + f];
      uint32_t w[8] = {0, 0, 0, 0, 0, 0, 0, 0};  // byte 31 stays 0 (pad)
      digitize_record(rec, [&](int pos, uint32_t d) { w[pos >> 2] |= d << ((pos & 3) * 8); });
      uint8_t *o = out + (base + tid) * 32;
      if (vec_out) {
        uint4 *o4 = reinterpret_cast<uint4 *>(o);
        __stcs(o4 + 0, make_uint4(w[0], w[1], w[2], w[3]));
        __stcs(o4 + 1, make_uint4(w[4], w[5], w[6], w[7]));
      } else {
#pragma unroll
        for (int b = 0; b < 32; ++b) o[b] = (uint8_t)(w[b >> 2] >> ((b & 3) * 8));
      }
    }
    __syncthreads();
  }
}

}  // namespace

cudaError_t launch_digitize(const lake_io_raw_t *raw, int64_t n, uint8_t *digits,
                            cudaStream_t s) {
  const int64_t nblocks = (n + kDigBlock - 1) / kDigBlock;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t grid = nblocks < (int64_t)sms * 8 ? nblocks : (int64_t)sms * 8;
  const bool vec_in = (reinterpret_cast<uintptr_t>(raw) & 15) == 0;
  const bool vec_out = (reinterpret_cast<uintptr_t>(digits) & 15) == 0;
  digitize_kernel<<<(unsigned)grid, kDigBlock, 0, s>>>(
      reinterpret_cast<const uint32_t *>(raw), n, digits, vec_in, vec_out);
  count_launch();
  return cudaGetLastError();
}

}  // namespace lake
