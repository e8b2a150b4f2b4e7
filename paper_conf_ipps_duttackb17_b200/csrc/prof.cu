// Launch counting and optional CUDA-event profiling of the library's kernels (ear_profile_* ABI).
#include <atomic>
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
