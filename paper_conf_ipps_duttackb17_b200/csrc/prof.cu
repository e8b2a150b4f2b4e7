// Launch counting and optional CUDA-event profiling of the library's kernels (ear_profile_* ABI).
#include <algorithm>
#include <atomic>
#include <cstring>
#include <mutex>
#include <vector>

#include "common.cuh"

namespace ear {
namespace {

struct Rec {
  int kind;
  cudaEvent_t e0, e1;
  double work;
};

std::atomic<long long> g_launches{0};
bool g_enabled = false;
std::mutex g_mu;
std::vector<Rec> g_pending;
std::vector<cudaEvent_t> g_pool;
ear_profile_t g_acc{};

cudaEvent_t get_event() {
  if (!g_pool.empty()) {
    cudaEvent_t e = g_pool.back();
    g_pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
  return e;
}

}  // namespace

void count_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

void prof_fw16_precheck() {
  std::lock_guard<std::mutex> lk(g_mu);
  g_acc.fw16_prechecked++;
}

void prof_fw16(bool used) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (used) g_acc.fw16_used++; else g_acc.fw16_fallbacks++;
}

int prof_begin(int kind, cudaStream_t s) {
  if (!g_enabled) return -1;
  std::lock_guard<std::mutex> lk(g_mu);
  Rec r{kind, get_event(), get_event(), 0.0};
  if (!r.e0 || !r.e1) return -1;
  cudaEventRecord(r.e0, s);
  g_pending.push_back(r);
  return (int)g_pending.size() - 1;
}

void prof_end(int slot, cudaStream_t s, double work) {
  if (slot < 0) return;
  std::lock_guard<std::mutex> lk(g_mu);
  if (slot >= (int)g_pending.size()) return;
  g_pending[slot].work = work;
  cudaEventRecord(g_pending[slot].e1, s);
}


// ---- small readbacks through mapped pinned memory (see Readback in common.cuh)
namespace {
constexpr size_t kStageBytes = 1 << 20;
struct Stage {
  char *h = nullptr;   // mapped pinned; the same pointer is valid on the device (UVA)
  size_t used = 0;
  bool failed = false;
};
thread_local Stage t_stage;

__global__ void k_readback(const unsigned char *__restrict__ src, unsigned char *__restrict__ dst, size_t bytes) {
  const bool w4 = ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst) | bytes) & 3) == 0;
  if (w4) {
    const uint32_t *s = reinterpret_cast<const uint32_t *>(src);
    uint32_t *d = reinterpret_cast<uint32_t *>(dst);
    for (size_t i = blockIdx.x * blockDim.x + threadIdx.x; i < bytes / 4; i += (size_t)gridDim.x * blockDim.x) d[i] = s[i];
  } else {
    for (size_t i = blockIdx.x * blockDim.x + threadIdx.x; i < bytes; i += (size_t)gridDim.x * blockDim.x) dst[i] = src[i];
  }
}

cudaError_t launch_readback(void *dst, const void *src, size_t bytes, cudaStream_t st) {
  const int grid = (int)std::min<size_t>(64, (bytes / 4 + 255) / 256 + 1);
  EAR_LAUNCH(k_readback, grid, 256, 0, st)(static_cast<const unsigned char *>(src), static_cast<unsigned char *>(dst), bytes);
  return cudaGetLastError();
}
}  // namespace

namespace {
__global__ void k_fill(unsigned char *__restrict__ dst, uint32_t word, size_t bytes) {
  const size_t stride = (size_t)gridDim.x * blockDim.x, t0 = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  const size_t mis = (16 - (reinterpret_cast<uintptr_t>(dst) & 15)) & 15, head = mis < bytes ? mis : bytes;
  for (size_t i = t0; i < head; i += stride) dst[i] = (unsigned char)word;
  uint4 *v = reinterpret_cast<uint4 *>(dst + head);
  const size_t nv = (bytes - head) / 16;
  for (size_t i = t0; i < nv; i += stride) v[i] = make_uint4(word, word, word, word);
  for (size_t i = head + nv * 16 + t0; i < bytes; i += stride) dst[i] = (unsigned char)word;
}
__global__ void k_copy_bytes(unsigned char *__restrict__ dst, const unsigned char *__restrict__ src, size_t bytes) {
  const size_t stride = (size_t)gridDim.x * blockDim.x, t0 = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  if (((reinterpret_cast<uintptr_t>(dst) | reinterpret_cast<uintptr_t>(src)) & 15) == 0) {
    const size_t nv = bytes / 16;
    for (size_t i = t0; i < nv; i += stride) reinterpret_cast<uint4 *>(dst)[i] = reinterpret_cast<const uint4 *>(src)[i];
    for (size_t i = nv * 16 + t0; i < bytes; i += stride) dst[i] = src[i];
  } else {
    for (size_t i = t0; i < bytes; i += stride) dst[i] = src[i];
  }
}
int fill_grid(size_t bytes) { return (int)std::max<size_t>(1, std::min<size_t>(148 * 8, (bytes / 16 + 255) / 256)); }
}  // namespace

cudaError_t dev_memset(void *dst, int value, size_t bytes, cudaStream_t st) {
  if (!bytes) return cudaSuccess;
  const uint32_t b = (uint32_t)(value & 0xFF);
  EAR_LAUNCH(k_fill, fill_grid(bytes), 256, 0, st)(static_cast<unsigned char *>(dst), b * 0x01010101u, bytes);
  return cudaGetLastError();
}

cudaError_t dev_copy(void *dst, const void *src, size_t bytes, cudaStream_t st) {
  if (!bytes) return cudaSuccess;
  EAR_LAUNCH(k_copy_bytes, fill_grid(bytes), 256, 0, st)(static_cast<unsigned char *>(dst),
                                                         static_cast<const unsigned char *>(src), bytes);
  return cudaGetLastError();
}

Readback::Readback(cudaStream_t st) : st_(st) {
  Stage &g = t_stage;
  if (!g.h && !g.failed && cudaHostAlloc((void **)&g.h, kStageBytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
    cudaGetLastError();
    g.h = nullptr;
    g.failed = true;
  }
  base_ = used_ = g.used;
}

Readback::~Readback() {
  if (pending_) cudaStreamSynchronize(st_);   // error path: let the stores land before the slots are reused
  if (t_stage.used == used_) t_stage.used = base_;   // release only when this object holds the top slots
}

cudaError_t Readback::get(void *h_dst, const void *d_src, size_t bytes) {
  if (bytes == 0) return cudaSuccess;
  Stage &g = t_stage;
  const size_t off = (std::max(used_, g.used) + 15) & ~size_t(15);   // above every live object's slots
  pending_ = true;
  if (!g.h || off + bytes > kStageBytes)   // no staging (or too big): the plain copy
    return cudaMemcpyAsync(h_dst, d_src, bytes, cudaMemcpyDeviceToHost, st_);
  cudaError_t e = launch_readback(g.h + off, d_src, bytes, st_);
  if (e != cudaSuccess) return e;
  slots_.push_back({h_dst, off, bytes});
  used_ = g.used = off + bytes;
  return cudaSuccess;
}

cudaError_t Readback::sync() {
  cudaError_t e = cudaStreamSynchronize(st_);
  pending_ = false;
  if (e == cudaSuccess)
    for (const Slot &s : slots_) std::memcpy(s.dst, t_stage.h + s.off, s.bytes);
  slots_.clear();
  if (t_stage.used == used_) t_stage.used = base_;
  used_ = base_;
  return e;
}

cudaError_t readback_direct(void *h_mapped, const void *d_src, size_t bytes, cudaStream_t st) {
  return bytes ? launch_readback(h_mapped, d_src, bytes, st) : cudaSuccess;
}

// ---- per-device helpers
int num_sms() {
  static std::atomic<int> cache[64];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 148;
  int v = cache[dev].load(std::memory_order_relaxed);
  if (v) return v;
  if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v < 1) v = 148;
  cache[dev].store(v, std::memory_order_relaxed);
  return v;
}

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) is per device and per kernel: raise it to the
// largest size requested so far for (device, kernel), under a lock
cudaError_t smem_attr(const void *kernel, int bytes) {
  static std::mutex mu;
  static std::vector<std::pair<std::pair<int, const void *>, int>> done;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> lk(mu);
  for (auto &d : done)
    if (d.first.first == dev && d.first.second == kernel) {
      if (d.second >= bytes) return cudaSuccess;
      e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
      if (e == cudaSuccess) d.second = bytes;
      return e;
    }
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess) done.push_back({{dev, kernel}, bytes});
  return e;
}

}  // namespace ear

using namespace ear;

extern "C" {

void ear_profile_enable(int32_t on) { g_enabled = on != 0; }

void ear_profile_reset(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  for (Rec &r : g_pending) {
    cudaEventSynchronize(r.e1);
    g_pool.push_back(r.e0);
    g_pool.push_back(r.e1);
  }
  g_pending.clear();
  g_acc = ear_profile_t{};
  g_launches.store(0);
}

ear_status_t ear_profile_read(ear_profile_t *out) {
  if (!out) return EAR_EINVAL;
  std::lock_guard<std::mutex> lk(g_mu);
  for (Rec &r : g_pending) {
    EAR_CUDA_TRY(cudaEventSynchronize(r.e1));
    float ms = 0.f;
    EAR_CUDA_TRY(cudaEventElapsedTime(&ms, r.e0, r.e1));
    switch (r.kind) {
      case PK_DECOMPOSE: g_acc.decompose_ms += ms; break;
      case PK_FW_INIT: g_acc.fw_init_ms += ms; break;
      case PK_FW_P1: g_acc.fw_phase1_ms += ms; g_acc.fw_phase1_launches++; break;
      case PK_FW_P2: g_acc.fw_phase2_ms += ms; g_acc.fw_phase2_launches++; g_acc.fw_phase2_minplus += r.work; break;
      case PK_FW_P3: g_acc.fw_phase3_ms += ms; g_acc.fw_phase3_launches++; g_acc.fw_phase3_minplus += r.work; break;
      case PK_COMM: g_acc.comm_ms += ms; break;
      case PK_EXPAND: g_acc.expand_ms += ms; g_acc.expand_launches++; g_acc.expand_bytes += r.work; break;
      case PK_SAME_CHAIN: g_acc.same_chain_ms += ms; break;
      case PK_SSSP: g_acc.sssp_ms += ms; g_acc.sssp_launches++; g_acc.sssp_arcs += r.work; break;
      case PK_BCC: g_acc.bcc_pieces_ms += ms; break;
      case PK_COMPOSE: g_acc.compose_ms += ms; g_acc.compose_bytes += r.work; break;
      case PK_FW_P3_16:
        g_acc.fw_phase3_ms += ms; g_acc.fw_phase3_launches++; g_acc.fw_phase3_minplus += r.work;
        g_acc.fw_phase3_16_ms += ms; g_acc.fw_phase3_16_minplus += r.work;
        break;
      case PK_FW16_CONV: g_acc.fw16_conv_ms += ms; break;
      case PK_FW_SIDE_P1: g_acc.fw_side_ms += ms; g_acc.fw_phase1_launches++; break;
      case PK_FW_SIDE_P2:
        g_acc.fw_side_ms += ms; g_acc.fw_phase2_launches++; g_acc.fw_phase2_minplus += r.work;
        break;
      case PK_REREDUCE: g_acc.rereduce_ms += ms; break;
      case PK_BCC_PREP: g_acc.bcc_prepare_ms += ms; break;
      case PK_EXPAND_D16: g_acc.expand_d16_ms += ms; break;
      case PK_PART: g_acc.part_ms += ms; break;
      case PK_PART_MP: g_acc.part_mp_ms += ms; g_acc.part_mp_launches++; g_acc.part_minplus += r.work; break;
      default: break;
    }
    g_pool.push_back(r.e0);
    g_pool.push_back(r.e1);
  }
  g_pending.clear();
  g_acc.launches = g_launches.load();
  *out = g_acc;
  return EAR_OK;
}

}  // extern "C"
