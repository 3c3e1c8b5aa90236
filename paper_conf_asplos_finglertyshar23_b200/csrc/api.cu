// api.cu — the C ABI (include/lake_linnos.h): argument validation, per-device model
// registry, weight-image preparation, dispatch to the kernels. See the header for the
// contract of every function; PAPER.md citations are there.
//
// Model registry: one DevModel table of LAKE_MAX_MODELS slots per CUDA device, mirrored
// on the host (for validation without a device round trip) and in device memory (for the
// multi-model kernels, which look a tile's model up by slot). A slot is the model_id — one
// model per block device, as the paper's per-device registries.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <atomic>
#include <cmath>
#include <cstring>
#include <memory>
#include <mutex>
#include <new>
#include <vector>

#include "lake_internal.h"

namespace lake {

static std::atomic<uint64_t> g_launches{0};
void count_launch(int k) { g_launches.fetch_add((uint64_t)k, std::memory_order_relaxed); }

namespace {

constexpr int kMaxDevices = 64;

struct ModelBufs {
  void *fp32 = nullptr;
  void *tc = nullptr;
};

struct DeviceState {
  bool init = false;
  DevModel host[LAKE_MAX_MODELS];
  ModelBufs bufs[LAKE_MAX_MODELS];
  DevModel *table = nullptr;  // device copy
};

std::mutex g_mu;
DeviceState *g_dev[kMaxDevices] = {nullptr};

// profiling of the main MLP kernel launches (bench roofline)
std::mutex g_prof_mu;
bool g_prof = false;
std::vector<std::pair<cudaEvent_t, cudaEvent_t>> g_prof_ev;
size_t g_prof_used = 0;

int nh_of(int32_t arch) { return arch + 1; }

// single-model FP32 calls with at most this many I/Os take the cluster small-batch kernel
// (measured device time vs the 16-row tile kernel: NN+1/NN+2 faster up to 64 rows; NN only
// up to 8 - its single 31-wide layer streams quickly through one CTA anyway)
inline int64_t fp32_small_max(int32_t arch) { return arch == LAKE_ARCH_NN ? 8 : LAKE_SERVER_MAX_BATCH; }

size_t blob_floats(int32_t arch) {
  switch (arch) {
    case LAKE_ARCH_NN: return 256 * 31 + 256 + 2 * 256 + 2;
    case LAKE_ARCH_NN1: return 256 * 31 + 256 + 256 * 256 + 256 + 2 * 256 + 2;
    case LAKE_ARCH_NN2: return 256 * 31 + 256 + 2 * (256 * 256 + 256) + 2 * 256 + 2;
    default: return 0;
  }
}

// Returns the state for `device`, creating the device table on first use.
// Caller holds g_mu and has made `device` current.
int get_state(int device, DeviceState **out) {
  if (device < 0 || device >= kMaxDevices) return LAKE_ERR_INVAL;
  DeviceState *st = g_dev[device];
  if (!st) {
    st = new (std::nothrow) DeviceState();
    if (!st) return LAKE_ERR_NOMEM;
    for (int i = 0; i < LAKE_MAX_MODELS; ++i) {
      std::memset(&st->host[i], 0, sizeof(DevModel));
      st->host[i].arch = -1;
    }
    g_dev[device] = st;
  }
  if (!st->init) {
    if (cudaMalloc(&st->table, sizeof(DevModel) * LAKE_MAX_MODELS) != cudaSuccess)
      return LAKE_ERR_NOMEM;
    if (cudaMemcpy(st->table, st->host, sizeof(DevModel) * LAKE_MAX_MODELS,
                   cudaMemcpyHostToDevice) != cudaSuccess)
      return LAKE_ERR_CUDA;
    st->init = true;
  }
  *out = st;
  return LAKE_OK;
}

// Permuted column position for the FP32 path (see lake_internal.h).
inline int perm_col(int j) {
  const int tc = j & 31, jj = j >> 5;
  return (jj >> 2) * 128 + tc * 4 + (jj & 3);
}

struct BlobView {
  const float *W[4];
  const float *b[4];
  int nh;
};

BlobView view_blob(int32_t arch, const float *blob) {
  BlobView v{};
  v.nh = nh_of(arch);
  const float *p = blob;
  v.W[0] = p; p += 256 * 31;
  v.b[0] = p; p += 256;
  for (int l = 1; l < v.nh; ++l) {
    v.W[l] = p; p += 256 * 256;
    v.b[l] = p; p += 256;
  }
  v.W[v.nh] = p; p += 2 * 256;
  v.b[v.nh] = p;
  return v;
}

// UMMA K-major SWIZZLE_NONE offset (bytes) of element (row r, k) in an R-row operand whose
// elements are `eb` bytes: a core matrix is 8 rows x 16 B (16/eb elements of K).
inline size_t umma_off(int r, int k, int R, int eb) {
  const int kc = 16 / eb;  // K elements per core matrix
  return (size_t)(k / kc) * (R * 16) + (size_t)r * 16 + (size_t)(k % kc) * eb;
}

// Operand encodings of one fp32 weight: 0 fp16, 1 bf16 (round to nearest even), 2 tf32
// (fp32 rounded to nearest even at 10 mantissa bits, low 13 bits zero; finite inputs only,
// checked at load).
inline uint32_t to_bits(float v, int prec) {
  if (prec == 0) {
    __half h = __float2half_rn(v);
    uint16_t u;
    std::memcpy(&u, &h, 2);
    return u;
  }
  if (prec == 1) {
    __nv_bfloat16 h = __float2bfloat16_rn(v);
    uint16_t u;
    std::memcpy(&u, &h, 2);
    return u;
  }
  uint32_t u;
  std::memcpy(&u, &v, 4);
  u += 0x0FFFu + ((u >> 13) & 1u);
  return u & ~0x1FFFu;
}

void build_tc_image(const BlobView &v, int prec, uint8_t *img /* 2 * bytes */, size_t bytes) {
  std::memset(img, 0, 2 * bytes);
  const int nh = v.nh;
  const int eb = (int)tc_elem_bytes(prec);
  for (int rank = 0; rank < 2; ++rank) {
    uint8_t *base = img + rank * bytes;
    auto put = [&](size_t off, float val) {
      const uint32_t u = to_bits(val, prec);
      std::memcpy(base + off, &u, eb);  // little endian: the low eb bytes
    };
    // layer 0 in the tensor-core K order: slot k holds digit tc_slot_digit(k) (lake_internal.h);
    // slot 31 holds b0, multiplied by the constant 1 the digitisers put in X's slot 31, so the
    // MMA adds layer 0's bias and its epilogue is only ReLU + rounding
    for (int n = 0; n < 128; ++n)
      for (int k = 0; k < kTcK0; ++k) {
        const int dgt = tc_slot_digit(k);
        const size_t row = (size_t)(rank * 128 + n);
        put(umma_off(n, k, 128, eb), dgt < 31 ? v.W[0][row * 31 + dgt] : v.b[0][row]);
      }
    for (int l = 1; l < nh; ++l) {
      const size_t o = tc_wh_off(l, prec);
      for (int n = 0; n < 128; ++n)
        for (int k = 0; k < 256; ++k)
          put(o + umma_off(n, k, 128, eb), v.W[l][(size_t)(rank * 128 + n) * 256 + k]);
      if (tc_bias_block_bytes(prec))  // bias block: K column 0 = b_l (the rest stays 0)
        for (int n = 0; n < 128; ++n)
          put(o + tc_wh_half_bytes(prec) + umma_off(n, 0, 128, eb), v.b[l][rank * 128 + n]);
    }
  }
}

// Release replaced model buffers: now, or once no persistent server runs (cudaFree would
// wait forever behind a resident server kernel; deferred.cu).
void retire_bufs(ModelBufs &b, int device) {
  release_device(b.fp32, device);
  release_device(b.tc, device);
  b.fp32 = b.tc = nullptr;
}

int cuda_status(cudaError_t e) {
  if (e == cudaSuccess) return LAKE_OK;
  if (e == cudaErrorMemoryAllocation) return LAKE_ERR_NOMEM;
  return LAKE_ERR_CUDA;
}

struct DeviceGuard {
  int prev = -1;
  bool ok = true;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) { ok = false; return; }
    if (prev != dev && cudaSetDevice(dev) != cudaSuccess) ok = false;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

// Look up a loaded model on the current device (validation for infer*).
int current_model(int32_t model_id, int *device, DevModel *out, const DevModel **table) {
  if (model_id < 0 || model_id >= LAKE_MAX_MODELS) return LAKE_ERR_NOMODEL;
  if (cudaGetDevice(device) != cudaSuccess) return LAKE_ERR_CUDA;
  std::lock_guard<std::mutex> lk(g_mu);
  if (*device < 0 || *device >= kMaxDevices || !g_dev[*device] || !g_dev[*device]->init)
    return LAKE_ERR_NOMODEL;
  const DevModel &m = g_dev[*device]->host[model_id];
  if (m.arch < 0) return LAKE_ERR_NOMODEL;
  *out = m;
  if (table) *table = g_dev[*device]->table;
  return LAKE_OK;
}

// *any: some model is loaded; *max_nh: the most hidden layers among the loaded models (the
// tensor-core kernel's SMEM layout for a multi-model call; tiles of a model loaded after this
// snapshot are clamped to it on the device, which keeps memory safe under that race).
// *has_nn: some loaded model is an NN (one hidden layer).
int current_table(int *device, const DevModel **table, int *any, int *max_nh = nullptr,
                  int *has_nn = nullptr) {
  if (cudaGetDevice(device) != cudaSuccess) return LAKE_ERR_CUDA;
  std::lock_guard<std::mutex> lk(g_mu);
  *any = 0;
  if (max_nh) *max_nh = 1;
  if (has_nn) *has_nn = 0;
  if (*device < 0 || *device >= kMaxDevices || !g_dev[*device] || !g_dev[*device]->init) {
    *table = nullptr;
    return LAKE_OK;
  }
  *table = g_dev[*device]->table;
  for (int i = 0; i < LAKE_MAX_MODELS; ++i)
    if (g_dev[*device]->host[i].arch >= 0) {
      *any = 1;
      if (max_nh && g_dev[*device]->host[i].nh > *max_nh) *max_nh = g_dev[*device]->host[i].nh;
      if (has_nn && g_dev[*device]->host[i].nh == 1) *has_nn = 1;
    }
  return LAKE_OK;
}

std::atomic<int64_t> g_auto_min[3] = {{LAKE_AUTO_TC_MIN_N_NN}, {LAKE_AUTO_TC_MIN_N_NN1},
                                      {LAKE_AUTO_TC_MIN_N_NN2}};

// arch < 0: unknown here (multi-model / host path before lookup) -> most conservative
int64_t auto_min(int32_t arch) {
  if (arch < 0 || arch > 2) {
    int64_t m = 0;
    for (int a = 0; a < 3; ++a) m = g_auto_min[a].load() > m ? g_auto_min[a].load() : m;
    return m;
  }
  return g_auto_min[arch].load();
}

int id_kind_of(uint32_t flags) { return (int)((flags & LAKE_IDS_MASK) >> 8); }
size_t id_bytes_of(uint32_t flags) { return (size_t)4 >> id_kind_of(flags); }

int check_flags(uint32_t flags, int64_t n, int *in_kind, int *prec, int32_t arch = -1) {
  if (flags & ~(uint32_t)(LAKE_IN_MASK | LAKE_PREC_MASK | LAKE_IDS_MASK)) return LAKE_ERR_INVAL;
  if ((flags & LAKE_IDS_MASK) == LAKE_IDS_MASK) return LAKE_ERR_INVAL;
  *in_kind = (int)(flags & LAKE_IN_MASK);
  const uint32_t p = flags & LAKE_PREC_MASK;
  switch (p) {
    case LAKE_PREC_FP32: *prec = -1; break;
    case LAKE_PREC_F16: *prec = 0; break;
    case LAKE_PREC_BF16: *prec = 1; break;
    case LAKE_PREC_TF32: *prec = 2; break;
    case LAKE_PREC_AUTO: *prec = (n >= auto_min(arch)) ? 0 : -1; break;
    default: return LAKE_ERR_INVAL;
  }
  return LAKE_OK;
}

int check_input_ptr(const void *in, int in_kind) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(in);
  if (in_kind == LAKE_IN_RAW) return (a & 3) ? LAKE_ERR_INVAL : LAKE_OK;
  return (a & 15) ? LAKE_ERR_INVAL : LAKE_OK;
}

struct ProfScope {
  cudaStream_t s;
  cudaEvent_t stop = nullptr;
  explicit ProfScope(cudaStream_t st) : s(st) {
    std::lock_guard<std::mutex> lk(g_prof_mu);
    if (!g_prof) return;
    if (g_prof_used == g_prof_ev.size()) {
      cudaEvent_t a, b;
      if (cudaEventCreate(&a) != cudaSuccess) return;
      if (cudaEventCreate(&b) != cudaSuccess) { cudaEventDestroy(a); return; }
      try {
        g_prof_ev.emplace_back(a, b);
      } catch (...) {  // out of host memory: this launch is simply not profiled
        cudaEventDestroy(a);
        cudaEventDestroy(b);
        return;
      }
    }
    auto &pr = g_prof_ev[g_prof_used++];
    cudaEventRecord(pr.first, s);
    stop = pr.second;
  }
  ~ProfScope() {
    if (stop) cudaEventRecord(stop, s);
  }
};

int launch_main(const void *in, int in_kind, int prec, const TileSched &ts, int nh_layout,
                uint8_t *decisions, float *logits, cudaStream_t s, int device) {
  cudaError_t e;
  {
    ProfScope ps(s);
    if (prec < 0)
      e = launch_mlp_fp32(in, in_kind, ts, decisions, logits, s, device);
    else
      e = launch_mlp_tc(in, in_kind, prec, ts, nh_layout, decisions, logits, s, device);
  }
  return cuda_status(e);
}

}  // namespace
}  // namespace lake

using namespace lake;

extern "C" {

size_t lake_linnos_blob_floats(int32_t arch) { return blob_floats(arch); }

int lake_linnos_load_weights(int32_t model_id, int32_t arch, const float *blob, size_t n_floats,
                             int32_t device) {
  if (model_id < 0 || model_id >= LAKE_MAX_MODELS) return LAKE_ERR_INVAL;
  if (arch < LAKE_ARCH_NN || arch > LAKE_ARCH_NN2) return LAKE_ERR_INVAL;
  if (!blob || n_floats != blob_floats(arch)) return LAKE_ERR_INVAL;
  if (device < 0 || device >= kMaxDevices) return LAKE_ERR_INVAL;
  for (size_t i = 0; i < n_floats; ++i)
    if (!std::isfinite(blob[i])) return LAKE_ERR_INVAL;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess) return LAKE_ERR_CUDA;
  if (device >= ndev) return LAKE_ERR_INVAL;

  const BlobView v = view_blob(arch, blob);
  const int nh = v.nh;
  // FP32 image: permuted W^T per hidden layer, biases, Wout, bout.
  const size_t f_w0 = 32 * 256, f_wh = 256 * 256;
  const size_t f_main = f_w0 + (nh - 1) * f_wh + nh * 256 + 2 * 256 + 4;
  const size_t f_total = f_main + (size_t)kServerCtas * kServerRankFloats;  // + cluster image
  std::unique_ptr<float[]> f(new (std::nothrow) float[f_total]());
  if (!f) return LAKE_ERR_NOMEM;
  size_t off_wt[kMaxHiddenLayers], off_b[kMaxHiddenLayers], off_wout, off_bout;
  {
    size_t p = 0;
    off_wt[0] = p;
    for (int k = 0; k < 31; ++k)
      for (int j = 0; j < 256; ++j) f[p + (size_t)k * 256 + perm_col(j)] = v.W[0][(size_t)j * 31 + k];
    p += f_w0;
    for (int l = 1; l < nh; ++l) {
      off_wt[l] = p;
      for (int k = 0; k < 256; ++k)
        for (int j = 0; j < 256; ++j)
          f[p + (size_t)k * 256 + perm_col(j)] = v.W[l][(size_t)j * 256 + k];
      p += f_wh;
    }
    for (int l = 0; l < nh; ++l) {
      off_b[l] = p;
      std::memcpy(&f[p], v.b[l], 256 * 4);
      p += 256;
    }
    off_wout = p;
    std::memcpy(&f[p], v.W[nh], 512 * 4);
    p += 512;
    off_bout = p;
    f[p] = v.b[nh][0];
    f[p + 1] = v.b[nh][1];
    // cluster image for server.cu: rank r holds output columns [32r, 32r + 32) of every layer
    for (int r = 0; r < kServerCtas; ++r) {
      float *q = &f[f_main + (size_t)r * kServerRankFloats];
      const int c0 = r * kServerSlice;
      for (int l = 0; l < nh; ++l)
        for (int j = 0; j < kServerSlice; ++j) q[l * kServerSlice + j] = v.b[l][c0 + j];
      q += kMaxHiddenLayers * kServerSlice;
      std::memcpy(q, v.W[nh], 512 * 4);
      q += 2 * 256;
      q[0] = v.b[nh][0];
      q[1] = v.b[nh][1];
      q += 4;
      for (int k = 0; k < 31; ++k)
        for (int j = 0; j < kServerSlice; ++j) q[k * kServerSlice + j] = v.W[0][(size_t)(c0 + j) * 31 + k];
      q += kInputs * kServerSlice;
      for (int l = 1; l < nh; ++l)
        for (int k = 0; k < 256; ++k)
          for (int j = 0; j < kServerSlice; ++j)
            q[(size_t)(l - 1) * 256 * kServerSlice + k * kServerSlice + j] =
                v.W[l][(size_t)(c0 + j) * 256 + k];
    }
  }
  // tensor-core images, [prec][rank]: fp16, bf16, tf32
  size_t tc_off[3], tc_total = 0;
  for (int p = 0; p < 3; ++p) {
    tc_off[p] = tc_total;
    tc_total += 2 * (size_t)tc_image_bytes(nh, p);
  }
  std::unique_ptr<uint8_t[]> img(new (std::nothrow) uint8_t[tc_total]);
  if (!img) return LAKE_ERR_NOMEM;
  for (int p = 0; p < 3; ++p) build_tc_image(v, p, img.get() + tc_off[p], tc_image_bytes(nh, p));

  std::lock_guard<std::mutex> lk(g_mu);
  DeviceGuard dg(device);
  if (!dg.ok) return LAKE_ERR_CUDA;
  DeviceState *st = nullptr;
  int rc = get_state(device, &st);
  if (rc != LAKE_OK) return rc;
  ModelBufs nb;
  if (cudaMalloc(&nb.fp32, f_total * 4) != cudaSuccess) return LAKE_ERR_NOMEM;
  if (cudaMalloc(&nb.tc, tc_total) != cudaSuccess) {
    retire_bufs(nb, device);
    return LAKE_ERR_NOMEM;
  }
  if (cudaMemcpy(nb.fp32, f.get(), f_total * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaMemcpy(nb.tc, img.get(), tc_total, cudaMemcpyHostToDevice) != cudaSuccess) {
    retire_bufs(nb, device);
    return LAKE_ERR_CUDA;
  }
  DevModel m;
  std::memset(&m, 0, sizeof(m));
  m.arch = arch;
  m.nh = nh;
  for (int p = 0; p < 3; ++p) m.tc_img[p] = static_cast<const uint8_t *>(nb.tc) + tc_off[p];
  const float *fb = static_cast<const float *>(nb.fp32);
  for (int l = 0; l < nh; ++l) {
    m.wt[l] = fb + off_wt[l];
    m.b[l] = fb + off_b[l];
  }
  m.wout = fb + off_wout;
  m.bout = fb + off_bout;
  m.srv = fb + f_main;  // 16-B aligned: f_main is a multiple of 4 floats
  // publish: device table entry, then host mirror; retire the previous buffers. (No
  // device-wide sync: in-flight work on this model is excluded by the header's contract.)
  if (cudaMemcpy(st->table + model_id, &m, sizeof(m), cudaMemcpyHostToDevice) != cudaSuccess) {
    retire_bufs(nb, device);
    return LAKE_ERR_CUDA;
  }
  retire_bufs(st->bufs[model_id], device);
  st->bufs[model_id] = nb;
  st->host[model_id] = m;
  return LAKE_OK;
}

int lake_linnos_unload(int32_t model_id, int32_t device) {
  if (model_id < 0 || model_id >= LAKE_MAX_MODELS) return LAKE_ERR_INVAL;
  if (device < 0 || device >= kMaxDevices) return LAKE_ERR_INVAL;
  std::lock_guard<std::mutex> lk(g_mu);
  DeviceState *st = g_dev[device];
  if (!st || !st->init || st->host[model_id].arch < 0) return LAKE_ERR_NOMODEL;
  DeviceGuard dg(device);
  if (!dg.ok) return LAKE_ERR_CUDA;
  DevModel m;
  std::memset(&m, 0, sizeof(m));
  m.arch = -1;
  if (cudaMemcpy(st->table + model_id, &m, sizeof(m), cudaMemcpyHostToDevice) != cudaSuccess)
    return LAKE_ERR_CUDA;
  retire_bufs(st->bufs[model_id], device);
  st->host[model_id] = m;
  return LAKE_OK;
}

int lake_linnos_model_arch(int32_t model_id, int32_t device, int32_t *arch_out) {
  if (!arch_out) return LAKE_ERR_INVAL;
  if (model_id < 0 || model_id >= LAKE_MAX_MODELS) return LAKE_ERR_NOMODEL;
  if (device < 0 || device >= kMaxDevices) return LAKE_ERR_INVAL;
  std::lock_guard<std::mutex> lk(g_mu);
  DeviceState *st = g_dev[device];
  if (!st || st->host[model_id].arch < 0) return LAKE_ERR_NOMODEL;
  *arch_out = st->host[model_id].arch;
  return LAKE_OK;
}

int lake_linnos_digitize(const lake_io_raw_t *raw, int64_t n, uint8_t *digits, void *stream) {
  if (n < 0) return LAKE_ERR_INVAL;
  if (n == 0) return LAKE_OK;
  if (!raw || !digits) return LAKE_ERR_INVAL;
  if (reinterpret_cast<uintptr_t>(raw) & 3) return LAKE_ERR_INVAL;
  return cuda_status(launch_digitize(raw, n, digits, static_cast<cudaStream_t>(stream)));
}

int lake_linnos_infer(const void *in, uint32_t flags, int64_t n, int32_t model_id,
                      uint8_t *decisions, float *logits, void *stream) {
  if (n < 0) return LAKE_ERR_INVAL;
  int in_kind, prec;
  int rc = check_flags(flags, n, &in_kind, &prec);
  if (rc != LAKE_OK) return rc;
  if (n == 0) return LAKE_OK;
  if (!in || !decisions) return LAKE_ERR_INVAL;
  if (check_input_ptr(in, in_kind) != LAKE_OK) return LAKE_ERR_INVAL;
  if (logits && (reinterpret_cast<uintptr_t>(logits) & 3)) return LAKE_ERR_INVAL;
  if (n > (int64_t)INT32_MAX) return LAKE_ERR_INVAL;
  int device;
  DevModel m;
  rc = current_model(model_id, &device, &m, nullptr);
  if (rc != LAKE_OK) return rc;
  if ((flags & LAKE_PREC_MASK) == LAKE_PREC_AUTO) check_flags(flags, n, &in_kind, &prec, m.arch);
  if (prec < 0 && n <= fp32_small_max(m.arch)) {
    // small batches: one 8-CTA cluster holds the weights across 8 SMs (server.cu), instead of
    // one CTA streaming every layer's W^T chunk by chunk (~1 L2 round trip per chunk)
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    ProfScope ps(s);
    return cuda_status(launch_fp32_small(m, in, in_kind, n, decisions, logits, s));
  }
  TileSched ts;
  std::memset(&ts, 0, sizeof(ts));
  const int rows = prec < 0 ? kF32TileM : kTcTileRows;
  ts.n_tiles = (n + rows - 1) / rows;
  ts.n = n;
  ts.model = m;
  return launch_main(in, in_kind, prec, ts, m.nh, decisions, logits,
                     static_cast<cudaStream_t>(stream), device);
}

int lake_linnos_auto_threshold(int32_t arch, int64_t *n_min_out) {
  if (arch < 0 || arch > 2 || !n_min_out) return LAKE_ERR_INVAL;
  *n_min_out = g_auto_min[arch].load();
  return LAKE_OK;
}

int lake_linnos_set_auto_threshold(int32_t arch, int64_t n_min) {
  if (arch < 0 || arch > 2 || n_min < 0) return LAKE_ERR_INVAL;
  g_auto_min[arch].store(n_min);
  return LAKE_OK;
}

size_t lake_linnos_workspace_bytes(int64_t n) {
  if (n < 0) return 0;
  return group_workspace_bytes(n);
}

int multi_group_impl(int64_t n, const void *model_ids, int id_kind, void *workspace,
                     size_t ws_bytes, void *stream, const void *in = nullptr, int in_kind = 0);
int multi_grouped_impl(const void *in, uint32_t flags, int64_t n, uint8_t *decisions,
                       float *logits, void *workspace, size_t ws_bytes, void *stream,
                       bool packed);

int lake_linnos_multi_group(int64_t n, const int32_t *model_ids, void *workspace,
                            size_t ws_bytes, void *stream) {
  return multi_group_impl(n, model_ids, 0, workspace, ws_bytes, stream);
}

int multi_group_impl(int64_t n, const void *model_ids, int id_kind, void *workspace,
                     size_t ws_bytes, void *stream, const void *in, int in_kind) {
  if (n < 0 || n > (int64_t)INT32_MAX) return LAKE_ERR_INVAL;
  if (n > 0 && !model_ids) return LAKE_ERR_INVAL;
  if (!workspace) return LAKE_ERR_INVAL;
  if (ws_bytes < group_workspace_bytes(n)) return LAKE_ERR_NOMEM;
  int device, any;
  const DevModel *table;
  int rc = current_table(&device, &table, &any);
  if (rc != LAKE_OK) return rc;
  if (!table) {
    // no model was ever loaded on this device: create the (empty) table so that every
    // id is reported unknown
    std::lock_guard<std::mutex> lk(g_mu);
    DeviceState *st;
    rc = get_state(device, &st);
    if (rc != LAKE_OK) return rc;
    table = st->table;
  }
  return cuda_status(
      launch_group(n, model_ids, id_kind, table, workspace, in, in_kind,
                   static_cast<cudaStream_t>(stream)));
}

int lake_linnos_multi_grouped(const void *in, uint32_t flags, int64_t n, uint8_t *decisions,
                              float *logits, void *workspace, size_t ws_bytes, void *stream) {
  return multi_grouped_impl(in, flags, n, decisions, logits, workspace, ws_bytes, stream, false);
}

int multi_grouped_impl(const void *in, uint32_t flags, int64_t n, uint8_t *decisions,
                       float *logits, void *workspace, size_t ws_bytes, void *stream,
                       bool packed) {
  if (n < 0 || n > (int64_t)INT32_MAX) return LAKE_ERR_INVAL;
  int in_kind, prec;
  int rc = check_flags(flags, n, &in_kind, &prec);
  if (rc != LAKE_OK) return rc;
  if (n == 0) return LAKE_OK;
  if (!in || !decisions || !workspace) return LAKE_ERR_INVAL;
  if (check_input_ptr(in, in_kind) != LAKE_OK) return LAKE_ERR_INVAL;
  if (ws_bytes < group_workspace_bytes(n)) return LAKE_ERR_NOMEM;
  int device, any, max_nh, has_nn;
  const DevModel *table;
  rc = current_table(&device, &table, &any, &max_nh, &has_nn);
  if (rc != LAKE_OK) return rc;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  cudaError_t e = launch_unknown_fill(workspace, n, decisions, logits, s);
  if (e != cudaSuccess) return cuda_status(e);
  if (!table || !any) return LAKE_OK;
  if (prec >= 0 && !packed) {  // grouped by a separate multi_group call: pack through perm
    e = launch_group_pack(workspace, n, in, in_kind, s);
    if (e != cudaSuccess) return cuda_status(e);
  }
  TileSched ts;
  std::memset(&ts, 0, sizeof(ts));
  group_sched(workspace, n, prec < 0 ? 0 : 1, table, &ts);
  if ((prec == 0 || prec == 1) && has_nn && max_nh > 1) {
    // NN and NN+1/NN+2 models loaded: the grouping put the NN tiles first; one kernel per
    // class (the NN kernel runs the output layer on the tensor cores, mlp_tc.cu)
    ts.part = 1;
    rc = launch_main(in, in_kind, prec, ts, 1, decisions, logits, s, device);
    if (rc != LAKE_OK) return rc;
    ts.part = 2;
  }
  return launch_main(in, in_kind, prec, ts, max_nh, decisions, logits, s, device);
}

int lake_linnos_infer_multi(const void *in, uint32_t flags, int64_t n, const int32_t *model_ids,
                            uint8_t *decisions, float *logits, void *workspace, size_t ws_bytes,
                            void *stream) {
  if (n < 0) return LAKE_ERR_INVAL;
  int in_kind, prec;
  int rc = check_flags(flags, n, &in_kind, &prec);
  if (rc != LAKE_OK) return rc;
  if (n == 0) return LAKE_OK;
  if (!in || !decisions || !model_ids || !workspace) return LAKE_ERR_INVAL;
  if (check_input_ptr(in, in_kind) != LAKE_OK) return LAKE_ERR_INVAL;
  // tensor-core paths: the scatter also packs every I/O's digit row in grouped order (read
  // in arrival order, coalesced), which the fused kernel then bulk-copies per tile
  rc = multi_group_impl(n, model_ids, id_kind_of(flags), workspace, ws_bytes, stream,
                        prec >= 0 ? in : nullptr, in_kind);
  if (rc != LAKE_OK) return rc;
  return multi_grouped_impl(in, flags & ~(uint32_t)LAKE_IDS_MASK, n, decisions, logits,
                            workspace, ws_bytes, stream, prec >= 0);
}

int lake_linnos_multi_status(const void *workspace, size_t ws_bytes, int64_t *n_unknown,
                             void *stream) {
  if (!workspace || !n_unknown) return LAKE_ERR_INVAL;
  (void)ws_bytes;
  GroupView v = group_view(const_cast<void *>(workspace), 0);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaMemcpyAsync(n_unknown, v.n_unknown, sizeof(int64_t),
                                  cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  return cuda_status(e);
}

}  // extern "C"

// ---- host-buffer path: chunked 3-stream pipeline ------------------------------------------
// chunk i: H2D (copy stream) -> group + fused kernel (caller's stream) -> D2H (copy-back
// stream), two staging slots, so the PCIe transfers of neighbouring chunks overlap compute.
namespace lake {
namespace {
#ifndef LAKE_HOST_CHUNK_LOG2
#define LAKE_HOST_CHUNK_LOG2 20
#endif
constexpr int64_t kHostChunk = (int64_t)1 << LAKE_HOST_CHUNK_LOG2;  // I/Os per pipelined chunk
constexpr int64_t kZeroCopyMax = 1 << 14;

// Device-accessible alias of a pinned, mapped host pointer (UVA), or nullptr.
void *mapped(const void *h) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, h) != cudaSuccess) {
    cudaGetLastError();  // pageable memory on older drivers reports an error: clear it
    return nullptr;
  }
  if (a.type != cudaMemoryTypeHost || a.devicePointer == nullptr) return nullptr;
  return a.devicePointer;
}

size_t a256(size_t x) { return (x + 255) & ~(size_t)255; }

struct SlotLayout {
  size_t in, ids, dec, log, ws, total;
};
SlotLayout slot_layout(int64_t chunk, size_t in_b) {
  SlotLayout L{};
  size_t o = 0;
  L.in = o; o += a256((size_t)chunk * in_b);
  L.ids = o; o += a256((size_t)chunk * 4);
  L.dec = o; o += a256((size_t)chunk);
  L.log = o; o += a256((size_t)chunk * 8);
  L.ws = o; o += a256(group_workspace_bytes(chunk));
  L.total = o;
  return L;
}

struct HostPipe {
  bool init = false;
  cudaStream_t h2d = nullptr, d2h = nullptr;
  cudaEvent_t start, in_ready[2], comp_done[2], out_done[2];
};
std::mutex g_pipe_mu;
HostPipe g_pipe[kMaxDevices];

int pipe_for(int device, HostPipe **out) {
  HostPipe &p = g_pipe[device];
  if (!p.init) {
    if (cudaStreamCreateWithFlags(&p.h2d, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&p.d2h, cudaStreamNonBlocking) != cudaSuccess)
      return LAKE_ERR_CUDA;
    if (cudaEventCreateWithFlags(&p.start, cudaEventDisableTiming) != cudaSuccess)
      return LAKE_ERR_CUDA;
    for (int i = 0; i < 2; ++i)
      if (cudaEventCreateWithFlags(&p.in_ready[i], cudaEventDisableTiming) != cudaSuccess ||
          cudaEventCreateWithFlags(&p.comp_done[i], cudaEventDisableTiming) != cudaSuccess ||
          cudaEventCreateWithFlags(&p.out_done[i], cudaEventDisableTiming) != cudaSuccess)
        return LAKE_ERR_CUDA;
    p.init = true;
  }
  *out = &p;
  return LAKE_OK;
}
}  // namespace
}  // namespace lake

extern "C" {

size_t lake_linnos_host_staging_bytes(int64_t n, uint32_t flags) {
  if (n < 0) return 0;
  const size_t in_b = (flags & LAKE_IN_MASK) == LAKE_IN_RAW ? 36 : 32;
  const int64_t chunk = n < kHostChunk ? (n > 0 ? n : 1) : kHostChunk;
  return 2 * slot_layout(chunk, in_b).total;
}

int lake_linnos_infer_host(const void *h_in, uint32_t flags, int64_t n, int32_t model_id,
                           const int32_t *h_model_ids, uint8_t *h_decisions, float *h_logits,
                           void *d_staging, size_t staging_bytes, void *stream) {
  if (n < 0) return LAKE_ERR_INVAL;
  int in_kind, prec;
  int rc = check_flags(flags, n, &in_kind, &prec);
  if (rc != LAKE_OK) return rc;
  if (n == 0) return LAKE_OK;
  if (!h_in || !h_decisions || !d_staging) return LAKE_ERR_INVAL;
  if (staging_bytes < lake_linnos_host_staging_bytes(n, flags)) return LAKE_ERR_NOMEM;
  int device;
  if (cudaGetDevice(&device) != cudaSuccess) return LAKE_ERR_CUDA;
  if (device < 0 || device >= kMaxDevices) return LAKE_ERR_INVAL;
  int32_t arch = -1;
  if (!h_model_ids) {  // validate the single model once, before any copy
    DevModel m;
    rc = current_model(model_id, &device, &m, nullptr);
    if (rc != LAKE_OK) return rc;
    arch = m.arch;
  }
  // AUTO decides on the whole batch, not per chunk
  if ((flags & LAKE_PREC_MASK) == LAKE_PREC_AUTO) {
    check_flags(flags, n, &in_kind, &prec, arch);
    flags = (flags & ~(uint32_t)LAKE_PREC_MASK) | (prec < 0 ? LAKE_PREC_FP32 : LAKE_PREC_F16);
  }
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const size_t in_b = in_kind == LAKE_IN_RAW ? 36 : 32;
  const size_t id_b = id_bytes_of(flags);
  const int64_t chunk = n < kHostChunk ? n : kHostChunk;
  const SlotLayout L = slot_layout(chunk, in_b);
  const int64_t nchunks = (n + chunk - 1) / chunk;
  uint8_t *base = static_cast<uint8_t *>(d_staging);
  if (n <= kZeroCopyMax) {
    // small batch: if every host buffer is pinned and mapped (UVA), the fused kernel reads
    // the records from and writes the decisions to host memory directly - no copy-engine
    // round trips (they, not the kernel, dominate the latency of a small batch)
    void *d_in = mapped(h_in), *d_dec = mapped(h_decisions);
    void *d_ids = h_model_ids ? mapped(h_model_ids) : nullptr;
    void *d_log = h_logits ? mapped(h_logits) : nullptr;
    if (d_in && d_dec && (!h_model_ids || d_ids) && (!h_logits || d_log)) {
      if (h_model_ids)
        rc = lake_linnos_infer_multi(d_in, flags, n, static_cast<int32_t *>(d_ids),
                                     static_cast<uint8_t *>(d_dec), static_cast<float *>(d_log),
                                     base + L.ws, L.total - L.ws, stream);
      else
        rc = lake_linnos_infer(d_in, flags, n, model_id, static_cast<uint8_t *>(d_dec),
                               static_cast<float *>(d_log), stream);
      if (rc != LAKE_OK) return rc;
      return cuda_status(cudaStreamSynchronize(s));
    }
  }
  if (nchunks == 1) {
    // one chunk: nothing to overlap, so stay on the caller's stream (no cross-stream hops)
    cudaError_t e = cudaMemcpyAsync(base + L.in, h_in, n * in_b, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess && h_model_ids)
      e = cudaMemcpyAsync(base + L.ids, h_model_ids, n * id_b, cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) return cuda_status(e);
    uint8_t *d_dec = base + L.dec;
    float *d_log = h_logits ? reinterpret_cast<float *>(base + L.log) : nullptr;
    if (h_model_ids)
      rc = lake_linnos_infer_multi(base + L.in, flags, n, reinterpret_cast<int32_t *>(base + L.ids),
                                   d_dec, d_log, base + L.ws, L.total - L.ws, stream);
    else
      rc = lake_linnos_infer(base + L.in, flags, n, model_id, d_dec, d_log, stream);
    if (rc != LAKE_OK) return rc;
    e = cudaMemcpyAsync(h_decisions, d_dec, n, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && h_logits)
      e = cudaMemcpyAsync(h_logits, d_log, n * 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    return cuda_status(e);
  }
  std::lock_guard<std::mutex> lk(g_pipe_mu);
  HostPipe *pp;
  rc = pipe_for(device, &pp);
  if (rc != LAKE_OK) return rc;
  // the staging slots must not be overwritten while earlier work on `s` still uses them
  cudaError_t e = cudaEventRecord(pp->start, s);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(pp->h2d, pp->start, 0);
  for (int64_t c = 0; c < nchunks && e == cudaSuccess; ++c) {
    const int slot = (int)(c & 1);
    uint8_t *sb = base + slot * L.total;
    const int64_t off = c * chunk;
    const int64_t cn = (n - off) < chunk ? (n - off) : chunk;
    if (c >= 2) e = cudaStreamWaitEvent(pp->h2d, pp->comp_done[slot], 0);  // input slot free
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(sb + L.in, static_cast<const uint8_t *>(h_in) + off * in_b, cn * in_b,
                          cudaMemcpyHostToDevice, pp->h2d);
    if (e == cudaSuccess && h_model_ids)
      e = cudaMemcpyAsync(sb + L.ids, reinterpret_cast<const uint8_t *>(h_model_ids) + off * id_b,
                          cn * id_b, cudaMemcpyHostToDevice, pp->h2d);
    if (e == cudaSuccess) e = cudaEventRecord(pp->in_ready[slot], pp->h2d);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(s, pp->in_ready[slot], 0);
    if (e == cudaSuccess && c >= 2) e = cudaStreamWaitEvent(s, pp->out_done[slot], 0);  // outputs read
    if (e != cudaSuccess) break;
    uint8_t *d_dec = sb + L.dec;
    float *d_log = h_logits ? reinterpret_cast<float *>(sb + L.log) : nullptr;
    if (h_model_ids)
      rc = lake_linnos_infer_multi(sb + L.in, flags, cn, reinterpret_cast<int32_t *>(sb + L.ids),
                                   d_dec, d_log, sb + L.ws, L.total - L.ws, stream);
    else
      rc = lake_linnos_infer(sb + L.in, flags, cn, model_id, d_dec, d_log, stream);
    if (rc != LAKE_OK) break;
    e = cudaEventRecord(pp->comp_done[slot], s);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(pp->d2h, pp->comp_done[slot], 0);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(h_decisions + off, d_dec, cn, cudaMemcpyDeviceToHost, pp->d2h);
    if (e == cudaSuccess && h_logits)
      e = cudaMemcpyAsync(h_logits + off * 2, d_log, cn * 8, cudaMemcpyDeviceToHost, pp->d2h);
    if (e == cudaSuccess) e = cudaEventRecord(pp->out_done[slot], pp->d2h);
  }
  cudaError_t e2 = cudaStreamSynchronize(pp->h2d);
  cudaError_t e3 = cudaStreamSynchronize(pp->d2h);
  cudaError_t e4 = cudaStreamSynchronize(s);
  if (rc != LAKE_OK) return rc;
  if (e == cudaSuccess) e = e2;
  if (e == cudaSuccess) e = e3;
  if (e == cudaSuccess) e = e4;
  return cuda_status(e);
}

size_t lake_linnos_capture_workspace_bytes(int64_t n) {
  if (n < 0 || n > (int64_t)INT32_MAX) return 0;
  return capture_workspace_bytes(n > 0 ? n : 1);
}

int lake_linnos_capture(const int64_t *arrival_ns, const int64_t *complete_ns,
                        const int32_t *device, int64_t n, lake_io_raw_t *raw_out,
                        void *workspace, size_t ws_bytes, void *stream) {
  if (n < 0 || n > (int64_t)INT32_MAX) return LAKE_ERR_INVAL;
  if (n == 0) return LAKE_OK;
  if (!arrival_ns || !complete_ns || !raw_out || !workspace) return LAKE_ERR_INVAL;
  if ((reinterpret_cast<uintptr_t>(arrival_ns) | reinterpret_cast<uintptr_t>(complete_ns)) & 7)
    return LAKE_ERR_INVAL;
  if (reinterpret_cast<uintptr_t>(raw_out) & 3) return LAKE_ERR_INVAL;
  if (device && (reinterpret_cast<uintptr_t>(device) & 3)) return LAKE_ERR_INVAL;
  return cuda_status(launch_capture(arrival_ns, complete_ns, device, n,
                                    reinterpret_cast<uint32_t *>(raw_out), workspace, ws_bytes,
                                    static_cast<cudaStream_t>(stream)));
}

int lake_linnos_server_start(int32_t model_id, lake_server_t **server_out) {
  if (!server_out) return LAKE_ERR_INVAL;
  int device;
  DevModel m;
  int rc = current_model(model_id, &device, &m, nullptr);
  if (rc != LAKE_OK) return rc;
  Server *s = nullptr;
  rc = server_start(m, device, &s);
  if (rc != LAKE_OK) return rc;
  *server_out = reinterpret_cast<lake_server_t *>(s);
  return LAKE_OK;
}

int lake_linnos_server_infer(lake_server_t *server, const lake_io_raw_t *h_raw, int32_t n,
                             uint8_t *h_decisions, float *h_logits) {
  if (!server || n < 0 || n > LAKE_SERVER_MAX_BATCH) return LAKE_ERR_INVAL;
  if (n == 0) return LAKE_OK;
  if (!h_raw || !h_decisions) return LAKE_ERR_INVAL;
  return server_infer(reinterpret_cast<Server *>(server), h_raw, n, h_decisions, h_logits);
}

int lake_linnos_server_stop(lake_server_t *server) {
  if (!server) return LAKE_ERR_INVAL;
  return server_stop(reinterpret_cast<Server *>(server));
}

uint64_t lake_linnos_launch_count(void) { return g_launches.load(); }
void lake_linnos_reset_launch_count(void) { g_launches.store(0); }

int lake_linnos_profile_enable(int enable) {
  std::lock_guard<std::mutex> lk(g_prof_mu);
  g_prof = enable != 0;
  g_prof_used = 0;
  return LAKE_OK;
}

int lake_linnos_profile_read(double *total_ms, int64_t *n_launches) {
  if (!total_ms || !n_launches) return LAKE_ERR_INVAL;
  std::lock_guard<std::mutex> lk(g_prof_mu);
  double tot = 0.0;
  for (size_t i = 0; i < g_prof_used; ++i) {
    cudaError_t e = cudaEventSynchronize(g_prof_ev[i].second);
    if (e != cudaSuccess) return cuda_status(e);
    float ms = 0.0f;
    e = cudaEventElapsedTime(&ms, g_prof_ev[i].first, g_prof_ev[i].second);
    if (e != cudaSuccess) return cuda_status(e);
    tot += ms;
  }
  *total_ms = tot;
  *n_launches = (int64_t)g_prof_used;
  g_prof_used = 0;
  return LAKE_OK;
}

const char *lake_linnos_strerror(int status) {
  switch (status) {
    case LAKE_OK: return "ok";
    case LAKE_ERR_INVAL: return "invalid argument";
    case LAKE_ERR_NOMODEL: return "model not loaded on the current device";
    case LAKE_ERR_CUDA: return "CUDA error";
    case LAKE_ERR_NOMEM: return "out of memory or workspace too small";
    case LAKE_ERR_UNSUPPORTED: return "unsupported in this build";
    default: return "unknown status";
  }
}

}  // extern "C"
