// server.cu — persistent resident-weights inference kernel with a host doorbell
// (SURVEY.md §8(f) NEXT-2). It attacks the paper's profitability problem (§4.2 P:583-603,
// Fig. 8): for small batches the cost is launch + copies + sync, not math.
//
// One cluster of kCtas CTAs stays resident. Each CTA keeps a 1/kCtas column slice of every
// hidden layer's weights in shared memory (NN+2's 561 KB of fp32 weights fit across 8 SMs),
// so nothing is reloaded per batch. The host writes the batch's raw records into a mailbox in
// mapped pinned memory and bumps a sequence number (the doorbell); CTA 0 polls it with
// system-scope acquire loads, the cluster digitises, evaluates the layers (each CTA its
// column slice, all-gathering activations through distributed shared memory), CTA 0 writes
// decisions / logits straight into the mailbox and publishes the sequence number back.
// Arithmetic is the FP32 path's strict order (reading R15): bit-exact with the oracle.
#include <atomic>
#include <cstring>
#include <new>

#include "digitize.cuh"
#include "lake_internal.h"
#include "lake_ptx.cuh"

namespace lake {
namespace {

constexpr int kCtas = 8;                       // cluster size (portable maximum)
constexpr int kSlice = kHidden / kCtas;        // output columns per CTA
constexpr int kThreadsS = 256;
constexpr uint32_t kStop = 0xFFFFFFFFu;
constexpr uint32_t kReady = 0xFFFFFFFEu;
constexpr int kActStride = kHidden + 4;  // 16-B aligned rows; 4-bank shift between rows

struct alignas(128) Mailbox {
  volatile uint32_t seq_in;   // host -> device: batch number (kStop = exit)
  volatile uint32_t n;
  uint32_t pad0[30];
  volatile uint32_t seq_out;  // device -> host: last completed batch
  uint32_t pad1[31];
  unsigned long long t[8];    // phase timestamps of the last batch (%globaltimer, ns)
};

// The first five members are, byte for byte, one rank's block of the model's cluster image
// (api.cu, DevModel::srv): one bulk copy of its used prefix loads a CTA's weights.
struct alignas(16) ServerSmem {
  float b[kMaxHiddenLayers][kSlice];
  float wout[2][kHidden];
  float bout[4];
  float w0[kInputs][kSlice];                 // W0^T slice
  float wh[kMaxHiddenLayers - 1][kHidden][kSlice];  // W_l^T slices, l = 1..nh-1
  unsigned long long wbar, wbar_pad;         // weight bulk-copy completion (16 B: act stays 16-B aligned)
  alignas(16) float act[2][LAKE_SERVER_MAX_BATCH][kActStride];  // all-gathered activations
  uint32_t rawbuf[LAKE_SERVER_MAX_BATCH * 9 + 4];    // CTA 0: the batch's raw records
  uint32_t seq;
  uint32_t n;
};

__device__ __forceinline__ uint32_t ld_acquire_sys(const volatile uint32_t *p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(volatile uint32_t *p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
#ifdef LAKE_SERVER_TIMES
#define SRV_T(i) (mb->t[i] = gtimer())
#else
#define SRV_T(i) ((void)0)
#endif
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void st_cluster_f32(uint32_t addr, float v) {
  asm volatile("st.shared::cluster.f32 [%0], %1;" :: "r"(addr), "f"(v) : "memory");
}
__device__ __forceinline__ void st_cluster_v4(uint32_t addr, float4 v) {
  asm volatile("st.shared::cluster.v4.f32 [%0], {%1,%2,%3,%4};"
               :: "r"(addr), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}
__device__ __forceinline__ uint4 ld_relaxed_sys_v4(const void *p) {
  uint4 v;
  asm volatile("ld.relaxed.sys.global.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
  return v;
}

// PERSISTENT: the doorbell server (this file's NEXT-2). !PERSISTENT: the same cluster
// evaluation launched once for one small batch already in device memory (n <= 64 raw records
// or digit rows), the FP32 path's small-batch kernel: the weights are spread over 8 SMs and
// fetched by all of them at once instead of streamed through one CTA layer by layer.
template <bool PERSISTENT, int IN_KIND>
__global__ void __cluster_dims__(kCtas, 1, 1) __launch_bounds__(kThreadsS, 1)
server_kernel(const __grid_constant__ DevModel model, Mailbox *mb, const uint32_t *raw,
              uint8_t *decisions, float *logits, uint32_t n_batch) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  ServerSmem &sm = *reinterpret_cast<ServerSmem *>(smem_raw);
  const int tid = threadIdx.x;
  const uint32_t rank = ptx::cluster_ctarank();
  const int col0 = rank * kSlice;
  const int nh = model.nh;
  // ---- resident weights: this CTA's block of the cluster image, one bulk copy (TMA)
  {
    const uint32_t wbar = ptx::smem_u32(&sm.wbar);
    const uint32_t bytes = server_block_bytes(nh);
    if (tid == 0) {
      ptx::mbar_init(wbar, 1);
      ptx::fence_mbar_init();
      ptx::mbar_arrive_expect_tx(wbar, bytes);
      ptx::bulk_g2s(ptx::smem_u32(&sm.b[0][0]), model.srv + (size_t)rank * kServerRankFloats,
                    bytes, wbar);
    }
    __syncthreads();
    ptx::mbar_wait(wbar, 0);
  }
  uint32_t act_remote[kCtas];  // shared::cluster address of act[0][0][0] in every CTA
  for (int c = 0; c < kCtas; ++c) act_remote[c] = ptx::mapa(ptx::smem_u32(&sm.act[0][0][0]), c);
  constexpr uint32_t kActBuf = LAKE_SERVER_MAX_BATCH * kActStride * 4;
  uint32_t last = 0;
  ptx::cluster_sync();
  if (PERSISTENT && rank == 0 && tid == 0) {  // weights resident: server_start may return
    __threadfence_system();
    st_release_sys(&mb->seq_out, kReady);
  }

  for (;;) {
    uint32_t seq0 = 0, n = n_batch;
    if constexpr (PERSISTENT) {
      // ---- doorbell: CTA 0 / thread 0 polls; everyone else sleeps in the cluster barrier
      if (rank == 0 && tid < 32) {
        if (tid == 0) {
          uint32_t s;
          while ((s = ld_acquire_sys(&mb->seq_in)) == last) __nanosleep(64);
          SRV_T(0);
          sm.seq = s;
          sm.n = mb->n;
        }
        __syncwarp();  // reconverge before the .aligned cluster barrier
      }
      ptx::cluster_sync();
      // every CTA reads seq/n from CTA 0's shared memory
      {
        const uint32_t a_seq = ptx::mapa(ptx::smem_u32(&sm.seq), 0);
        const uint32_t a_n = ptx::mapa(ptx::smem_u32(&sm.n), 0);
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(seq0) : "r"(a_seq) : "memory");
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(n) : "r"(a_n) : "memory");
      }
      if (seq0 == kStop) break;
      last = seq0;
    }
    if (n > LAKE_SERVER_MAX_BATCH) n = LAKE_SERVER_MAX_BATCH;
    // ---- CTA 0 fetches the batch once (persistent: 16-byte system-scope loads from the
    // mailbox), digitises it and broadcasts the digit rows into every CTA's act[0]
    if (rank == 0) {
      if constexpr (PERSISTENT) {  // the mailbox is padded: whole 16-B vectors
        const int n16 = ((int)n * 36 + 15) / 16;
        for (int i = tid; i < n16; i += kThreadsS)
          reinterpret_cast<uint4 *>(sm.rawbuf)[i] =
              ld_relaxed_sys_v4(reinterpret_cast<const uint4 *>(raw) + i);
      } else {  // caller's device buffer: exactly its n rows, 4-B loads
        const int nw = (int)n * (IN_KIND == LAKE_IN_RAW ? 9 : 8);
        for (int i = tid; i < nw; i += kThreadsS) sm.rawbuf[i] = __ldg(raw + i);
      }
      __syncthreads();
      if (tid < (int)n) {
        float dg[32];
        dg[31] = 0.0f;
        if constexpr (IN_KIND == LAKE_IN_RAW) {
          uint32_t rec[9];
#pragma unroll
          for (int f = 0; f < 9; ++f) rec[f] = sm.rawbuf[tid * 9 + f];
          digitize_record(rec, [&](int pos, uint32_t d) { dg[pos] = (float)d; });
        } else {
#pragma unroll
          for (int k = 0; k < 31; ++k)
            dg[k] = (float)((sm.rawbuf[tid * 8 + (k >> 2)] >> ((k & 3) * 8)) & 0xFFu);
        }
        const uint32_t off = (uint32_t)(tid * kActStride) * 4;
#pragma unroll
        for (int c = 0; c < kCtas; ++c)
#pragma unroll
          for (int q4 = 0; q4 < 8; ++q4)
            st_cluster_v4(act_remote[c] + off + q4 * 16,
                          make_float4(dg[4 * q4], dg[4 * q4 + 1], dg[4 * q4 + 2], dg[4 * q4 + 3]));
      }
    }
    ptx::cluster_sync();
    if (rank == 0 && tid == 0) SRV_T(1);
    // ---- hidden layers: this CTA's columns, all-gathered into every CTA. Thread t owns
    // columns 4*(t%8).. of the slice for rows t/8 and t/8 + 32 (strict k order per output)
    for (int l = 0; l < nh; ++l) {
      const float (*ain)[kActStride] = sm.act[l & 1];
      const uint32_t out_off = ((l + 1) & 1) * kActBuf;
      const int K = l == 0 ? kInputs : kHidden;
      const int cg = tid & 7, r0 = tid >> 3;
      const float (*w)[kSlice] = l == 0 ? sm.w0 : sm.wh[l - 1];
      if (r0 < (int)n) {
        const bool two = r0 + 32 < (int)n;
        float a0[4] = {0.0f, 0.0f, 0.0f, 0.0f}, a1[4] = {0.0f, 0.0f, 0.0f, 0.0f};
#pragma unroll 4
        for (int k = 0; k < K; ++k) {
          const float4 wk = *reinterpret_cast<const float4 *>(&w[k][cg * 4]);
          const float x0 = ain[r0][k];
          a0[0] = __fmaf_rn(x0, wk.x, a0[0]);
          a0[1] = __fmaf_rn(x0, wk.y, a0[1]);
          a0[2] = __fmaf_rn(x0, wk.z, a0[2]);
          a0[3] = __fmaf_rn(x0, wk.w, a0[3]);
          if (two) {
            const float x1 = ain[r0 + 32][k];
            a1[0] = __fmaf_rn(x1, wk.x, a1[0]);
            a1[1] = __fmaf_rn(x1, wk.y, a1[1]);
            a1[2] = __fmaf_rn(x1, wk.z, a1[2]);
            a1[3] = __fmaf_rn(x1, wk.w, a1[3]);
          }
        }
        float h0[4], h1[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float bj = sm.b[l][cg * 4 + e];
          const float z0 = __fadd_rn(a0[e], bj), z1 = __fadd_rn(a1[e], bj);
          h0[e] = (z0 > 0.0f) ? z0 : 0.0f;
          h1[e] = (z1 > 0.0f) ? z1 : 0.0f;
        }
        const uint32_t o0 = out_off + (uint32_t)(r0 * kActStride + col0 + cg * 4) * 4;
        const uint32_t o1 = o0 + 32u * kActStride * 4;
#pragma unroll
        for (int c = 0; c < kCtas; ++c) {
          st_cluster_v4(act_remote[c] + o0, make_float4(h0[0], h0[1], h0[2], h0[3]));
          if (two) st_cluster_v4(act_remote[c] + o1, make_float4(h1[0], h1[1], h1[2], h1[3]));
        }
      }
      ptx::cluster_sync();
      if (rank == 0 && tid == 0) SRV_T(2 + l);
    }
    // ---- output layer + decision (CTA 0), straight into the host mailbox
    if (rank == 0) {
      const float (*h)[kActStride] = sm.act[nh & 1];
      if (tid < 2 * LAKE_SERVER_MAX_BATCH) {  // whole warps take part in the shuffle
        const int r = tid >> 1, c = tid & 1;
        float z = 0.0f;
        if (r < (int)n) {
          float acc = 0.0f;
          for (int k = 0; k < kHidden; ++k) acc = __fmaf_rn(h[r][k], sm.wout[c][k], acc);
          z = __fadd_rn(acc, sm.bout[c]);
        }
        const float other = __shfl_xor_sync(0xffffffffu, z, 1);
        if (r < (int)n) {
          if (logits) logits[r * 2 + c] = z;
          if (c == 0) decisions[r] = (other > z) ? 1 : 0;  // logit1 > logit0; ties/NaN -> 0
        }
      }
      if constexpr (PERSISTENT) {
        __syncthreads();
        if (tid == 0) {
          SRV_T(5);
          __threadfence_system();
          SRV_T(6);
          st_release_sys(&mb->seq_out, seq0);
        }
        __syncwarp();
      }
    }
    if constexpr (!PERSISTENT) break;
  }
  ptx::cluster_sync();  // no CTA leaves while a peer may still read its shared memory
}

template <int IN_KIND>
cudaError_t small_launch(const DevModel &m, const void *in, int64_t n, uint8_t *dec, float *logits,
                         cudaStream_t st) {
  static std::atomic<bool> attr_set[64];  // per device; a race repeats the attribute call
  int dev = 0;
  cudaGetDevice(&dev);
  if (!attr_set[dev & 63].load(std::memory_order_acquire)) {
    cudaError_t e = cudaFuncSetAttribute(server_kernel<false, IN_KIND>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)sizeof(ServerSmem));
    if (e != cudaSuccess) return e;
    attr_set[dev & 63].store(true, std::memory_order_release);
  }
  server_kernel<false, IN_KIND><<<kCtas, kThreadsS, sizeof(ServerSmem), st>>>(
      m, nullptr, static_cast<const uint32_t *>(in), dec, logits, (uint32_t)n);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_fp32_small(const DevModel &m, const void *in, int in_kind, int64_t n,
                              uint8_t *dec, float *logits, cudaStream_t s) {
  count_launch();
  return in_kind == LAKE_IN_RAW ? small_launch<LAKE_IN_RAW>(m, in, n, dec, logits, s)
                                : small_launch<LAKE_IN_DIGITS>(m, in, n, dec, logits, s);
}

struct Server {
  int device = 0;
  int32_t model_id = 0;
  uint8_t *host = nullptr;     // mapped pinned block: mailbox | raw | decisions | logits
  Mailbox *mb = nullptr;
  uint32_t *raw = nullptr;
  uint8_t *dec = nullptr;
  float *log = nullptr;
  cudaStream_t stream = nullptr;
  uint32_t seq = 0;
};

size_t server_smem_bytes() { return sizeof(ServerSmem); }
int server_device(const Server *s) { return s->device; }

int server_start(const DevModel &m, int device, Server **out) {
  Server *s = new (std::nothrow) Server();
  if (!s) return LAKE_ERR_NOMEM;
  s->device = device;
  const size_t bytes = sizeof(Mailbox) + LAKE_SERVER_MAX_BATCH * (36 + 1 + 8) + 256;
  if (cudaHostAlloc(&s->host, bytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
    delete s;
    return LAKE_ERR_NOMEM;
  }
  std::memset(s->host, 0, bytes);
  s->mb = reinterpret_cast<Mailbox *>(s->host);
  s->raw = reinterpret_cast<uint32_t *>(s->host + sizeof(Mailbox));
  s->dec = s->host + sizeof(Mailbox) + LAKE_SERVER_MAX_BATCH * 36;
  s->log = reinterpret_cast<float *>(s->host + sizeof(Mailbox) + LAKE_SERVER_MAX_BATCH * 40);
  void *d_host = nullptr;
  cudaError_t e = cudaHostGetDevicePointer(&d_host, s->host, 0);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&s->stream, cudaStreamNonBlocking);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(server_kernel<true, LAKE_IN_RAW>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(ServerSmem));
  if (e != cudaSuccess) {
    release_host(s->host);
    delete s;
    return LAKE_ERR_CUDA;
  }
  uint8_t *d = static_cast<uint8_t *>(d_host);
  servers_started();  // from here on, library frees defer until the last server stops
  server_kernel<true, LAKE_IN_RAW><<<kCtas, kThreadsS, sizeof(ServerSmem), s->stream>>>(
      m, reinterpret_cast<Mailbox *>(d), reinterpret_cast<const uint32_t *>(d + sizeof(Mailbox)),
      d + sizeof(Mailbox) + LAKE_SERVER_MAX_BATCH * 36,
      reinterpret_cast<float *>(d + sizeof(Mailbox) + LAKE_SERVER_MAX_BATCH * 40), 0);
  count_launch();
  e = cudaGetLastError();
  // wait until the weights are resident (the model may be unloaded right after we return)
  while (e == cudaSuccess && s->mb->seq_out != kReady) {
    const cudaError_t q = cudaStreamQuery(s->stream);
    if (q != cudaErrorNotReady) e = (q == cudaSuccess) ? cudaErrorLaunchFailure : q;
  }
  if (e != cudaSuccess) {
    cudaStreamDestroy(s->stream);
    release_host(s->host);
    delete s;
    servers_stopped();
    return LAKE_ERR_CUDA;
  }
  *out = s;
  return LAKE_OK;
}

int server_infer(Server *s, const lake_io_raw_t *raw, int32_t n, uint8_t *dec, float *logits) {
  std::memcpy(s->raw, raw, (size_t)n * 36);
  s->mb->n = (uint32_t)n;
  if (++s->seq >= kReady) s->seq = 1;
  const uint32_t seq = s->seq;
  __sync_synchronize();  // records and n visible before the doorbell
  s->mb->seq_in = seq;
  // spin on the device's completion flag (a few microseconds)
  long spins = 0;
  while (s->mb->seq_out != seq) {
#if defined(__x86_64__)
    __builtin_ia32_pause();
#endif
    if (++spins > (1L << 34)) return LAKE_ERR_CUDA;
    if ((spins & 0xFFFFF) == 0 && cudaStreamQuery(s->stream) != cudaErrorNotReady)
      return LAKE_ERR_CUDA;  // the server kernel is gone
  }
  __sync_synchronize();
  std::memcpy(dec, s->dec, (size_t)n);
  if (logits) std::memcpy(logits, s->log, (size_t)n * 8);
  return LAKE_OK;
}

int server_stop(Server *s) {
  __sync_synchronize();
  s->mb->seq_in = kStop;
  cudaError_t e = cudaStreamSynchronize(s->stream);  // this server's kernel only
  cudaStreamDestroy(s->stream);
  release_host(s->host);  // parked while other servers still run (deferred.cu)
  delete s;
  servers_stopped();
  return e == cudaSuccess ? LAKE_OK : LAKE_ERR_CUDA;
}

}  // namespace lake

// development hook (not part of the ABI): phase timestamps of the server's last batch
// (recorded only when built with -DLAKE_SERVER_TIMES)
extern "C" void lake_debug_server_times(void *server, unsigned long long *out) {
  lake::Server *s = reinterpret_cast<lake::Server *>(server);
  for (int i = 0; i < 8; ++i) out[i] = s->mb->t[i];
}
