// Peer-memory transport of the row-block-sharded FW: one process per GPU (several
// processes may share one GPU), each rank owning a WINDOW -- one cudaMalloc allocation exported by CUDA
// IPC and mapped by every other rank (over NVLink/NVSwitch between GPUs, plain device memory on the same
// GPU).  Ranks write into each other's windows with ordinary kernel stores and publish progress through
// 64-bit flag slots (system-scope release stores); a rank waits for a flag in its OWN window with
// cuStreamWaitValue64 (stream-ordered, no SM held while waiting).  The host plumbing -- exchanging the
// IPC handles -- goes through the caller's all-gather callback (torch.distributed in the Python
// binding), collectively, at init and whenever a call needs a larger window.
//
// Window layout (identical on every rank, sized for the largest Np seen so far):
//   [0, 64 KB)      flag slots, uint64: PIECES[64] (round pieces delivered by rank r), TILE[64]
//                   (closed pivot tile pushed by its owner), BARRIER[64], CHECK[64]
//   L[2]            128 x Np elements each (round parity): the pivot row block being assembled for
//                   phase 2 -- each rank's own pieces, and the pivot tile pushed in by its owner
//   stage[3]        128 x Np elements each (round mod 3): the complete phase-2-updated pivot row block,
//                   written piece by piece by every rank (the per-round "broadcast" of the pieces)
//   region          nown x 128 x Np int32: this rank's owned tile rows after the FW, read by every
//                   peer for the final all-gather of D
#include <cuda.h>
#include <cudaTypedefs.h>

#include <cstring>
#include <mutex>

#include "common.cuh"

namespace ear {
namespace {

constexpr size_t kFlagBytes = 64 << 10;

PFN_cuStreamWaitValue64_v11070 g_wait64 = nullptr;
std::once_flag g_wait_once;

ear_status_t wait_fn() {
  std::call_once(g_wait_once, [] {
    cudaDriverEntryPointQueryResult q;
    void *fn = nullptr;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue64", &fn, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      g_wait64 = (PFN_cuStreamWaitValue64_v11070)fn;
    cudaGetLastError();
  });
  if (!g_wait64) {
    set_error("comm: cuStreamWaitValue64 unavailable");
    return EAR_ECUDA;
  }
  return EAR_OK;
}

// value -> slot [base + rank] of every destination window (release at system scope: the stores that
// precede it in stream order are visible to a peer that observes the flag)
__global__ void k_signal(PeerPtrs dst, int32_t slot, uint64_t value) {
  __threadfence_system();
  for (int p = threadIdx.x; p < dst.n; p += blockDim.x) {
    uint64_t *f = reinterpret_cast<uint64_t *>(dst.p[p]) + slot;
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(value) : "memory");
  }
}

}  // namespace

size_t comm_win_bytes(int32_t Np, int32_t nown) {
  const size_t blk = (size_t)TILE * Np * sizeof(int32_t);
  return kFlagBytes + 2 * blk + 3 * blk + (size_t)nown * blk;
}

char *comm_L(ear_comm_s *c, int p, int b) {
  return c->peer[p] + kFlagBytes + (size_t)b * TILE * c->np * sizeof(int32_t);
}
char *comm_stage(ear_comm_s *c, int p, int b) {
  return c->peer[p] + kFlagBytes + (size_t)(2 + b) * TILE * c->np * sizeof(int32_t);
}
int32_t *comm_region(ear_comm_s *c, int p) {
  return reinterpret_cast<int32_t *>(c->peer[p] + kFlagBytes + (size_t)5 * TILE * c->np * sizeof(int32_t));
}
PeerPtrs comm_flags_all(ear_comm_s *c) {
  PeerPtrs d{};
  d.n = c->nranks;
  for (int p = 0; p < c->nranks; ++p) d.p[p] = c->peer[p];
  return d;
}

static ear_status_t host_allgather(ear_comm_s *c, const void *send, void *recv, int64_t bytes) {
  if (c->nranks == 1) {
    memcpy(recv, send, (size_t)bytes);
    return EAR_OK;
  }
  if (!c->allgather || c->allgather(send, recv, bytes, c->ctx) != 0) {
    set_error("comm: the all-gather callback failed");
    return EAR_ENCCL;
  }
  return EAR_OK;
}

static void release_window(ear_comm_s *c) {
  for (int p = 0; p < c->nranks; ++p)
    if (p != c->rank && c->peer[p]) cudaIpcCloseMemHandle(c->peer[p]);
  if (c->win) cudaFree(c->win);
  c->win = nullptr;
  c->win_bytes = 0;
  for (int p = 0; p < c->nranks; ++p) c->peer[p] = nullptr;
  cudaGetLastError();
}

// Collective: make every rank's window hold the layout for (Np, nown).  Every rank passes the same
// sizes (nown is Np / 128 / P for every rank).  Grows only; a regrow synchronises `st`, agrees through
// the callback (no peer still reads the old window: each has synchronised too), and re-exchanges the
// IPC handles.  The flag sequences restart at zero with a new window.
ear_status_t comm_reserve(ear_comm_s *c, int32_t Np, int32_t nown, cudaStream_t st) {
  EAR_TRY(wait_fn());
  const size_t need = comm_win_bytes(Np, nown);
  int32_t want = (int32_t)(need > c->win_bytes), any = 0;
  std::vector<int32_t> all(c->nranks);
  EAR_TRY(host_allgather(c, &want, all.data(), sizeof(int32_t)));
  for (int32_t v : all) any |= v;
  if (any) {
    EAR_CUDA_TRY(cudaStreamSynchronize(st));
    EAR_CUDA_TRY(cudaDeviceSynchronize());
    uint8_t dummy = 0;
    std::vector<uint8_t> sink(c->nranks);
    EAR_TRY(host_allgather(c, &dummy, sink.data(), 1));   // every rank is past its last use of the old windows
    release_window(c);
    const size_t bytes = std::max(need, c->win_bytes) + (need >> 3);
    EAR_CUDA_TRY(cudaMalloc((void **)&c->win, bytes));
    EAR_CUDA_TRY(cudaMemset(c->win, 0, kFlagBytes));
    EAR_CUDA_TRY(cudaDeviceSynchronize());
    c->win_bytes = bytes;
    c->seq_pieces = c->seq_tile = c->seq_barrier = c->seq_check = 0;
    cudaIpcMemHandle_t h;
    if (c->nranks > 1) EAR_CUDA_TRY(cudaIpcGetMemHandle(&h, c->win));
    std::vector<cudaIpcMemHandle_t> hs(c->nranks);
    EAR_TRY(host_allgather(c, &h, hs.data(), sizeof(h)));
    std::vector<uint64_t> sizes(c->nranks);
    uint64_t b64 = bytes;
    EAR_TRY(host_allgather(c, &b64, sizes.data(), sizeof(b64)));
    for (int p = 0; p < c->nranks; ++p) {
      if (sizes[p] != bytes) { set_error("comm_reserve: ranks disagree on the window size"); return EAR_EINVAL; }
      if (p == c->rank) { c->peer[p] = c->win; continue; }
      EAR_CUDA_TRY(cudaIpcOpenMemHandle((void **)&c->peer[p], hs[p], cudaIpcMemLazyEnablePeerAccess));
    }
  }
  c->np = Np;
  return EAR_OK;
}

// flag slot `slot + rank` := value in every rank's window (after the stream's preceding work)
ear_status_t comm_signal(ear_comm_s *c, int32_t slot, uint64_t value, cudaStream_t st) {
  EAR_LAUNCH(k_signal, 1, 32, 0, st)(comm_flags_all(c), slot + c->rank, value);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// the stream waits until every slot [slot, slot + P) of this rank's window holds >= value
ear_status_t comm_wait(ear_comm_s *c, int32_t slot, uint64_t value, cudaStream_t st) {
  EAR_TRY(wait_fn());
  uint64_t *f = reinterpret_cast<uint64_t *>(c->win) + slot;
  for (int p = 0; p < c->nranks; ++p) {
    CUresult r = g_wait64((CUstream)st, (CUdeviceptr)(f + p), (cuuint64_t)value, CU_STREAM_WAIT_VALUE_GEQ);
    if (r != CUDA_SUCCESS) {
      set_error("comm_wait: cuStreamWaitValue64 failed (%d)", (int)r);
      return EAR_ECUDA;
    }
  }
  return EAR_OK;
}

// the stream waits for ONE slot of this rank's window
ear_status_t comm_wait_one(ear_comm_s *c, int32_t slot, uint64_t value, cudaStream_t st) {
  EAR_TRY(wait_fn());
  uint64_t *f = reinterpret_cast<uint64_t *>(c->win) + slot;
  CUresult r = g_wait64((CUstream)st, (CUdeviceptr)f, (cuuint64_t)value, CU_STREAM_WAIT_VALUE_GEQ);
  if (r != CUDA_SUCCESS) {
    set_error("comm_wait: cuStreamWaitValue64 failed (%d)", (int)r);
    return EAR_ECUDA;
  }
  return EAR_OK;
}

// stream-ordered barrier over the ranks: every rank's preceding work on `st` is done (and its
// stores visible) before any rank's following work on `st` starts
ear_status_t comm_barrier(ear_comm_s *c, cudaStream_t st) {
  const uint64_t v = ++c->seq_barrier;
  EAR_TRY(comm_signal(c, SLOT_BARRIER, v, st));
  return comm_wait(c, SLOT_BARRIER, v, st);
}

}  // namespace ear

extern "C" {

ear_status_t ear_comm_init(int32_t nranks, int32_t rank, ear_allgather_fn allgather, void *ctx, ear_comm_t *out) {
  if (!out || nranks < 1 || nranks > EAR_MAX_RANKS || rank < 0 || rank >= nranks || (nranks > 1 && !allgather)) {
    ear::set_error("ear_comm_init: bad arguments (nranks 1..%d, rank in [0,nranks), allgather needed for nranks > 1)",
                   EAR_MAX_RANKS);
    return EAR_EINVAL;
  }
  ear_comm_s *cm = new ear_comm_s;
  cm->nranks = nranks;
  cm->rank = rank;
  cm->allgather = allgather;
  cm->ctx = ctx;
  cudaGetDevice(&cm->device);
  // agree on the rank layout once (every rank must have called with the same nranks)
  int32_t mine[2] = {nranks, rank};
  std::vector<int32_t> all(2 * (size_t)nranks);
  ear_status_t s = ear::host_allgather(cm, mine, all.data(), sizeof(mine));
  for (int p = 0; p < nranks && s == EAR_OK; ++p)
    if (all[2 * p] != nranks || all[2 * p + 1] != p) {
      ear::set_error("ear_comm_init: rank %d reports (nranks %d, rank %d)", p, all[2 * p], all[2 * p + 1]);
      s = EAR_EINVAL;
    }
  if (s != EAR_OK) {
    delete cm;
    return s;
  }
  *out = cm;
  return EAR_OK;
}

ear_status_t ear_comm_info(ear_comm_t comm, int32_t *nranks, int32_t *rank) {
  if (!comm) {
    if (nranks) *nranks = 1;
    if (rank) *rank = 0;
    return EAR_OK;
  }
  if (nranks) *nranks = comm->nranks;
  if (rank) *rank = comm->rank;
  return EAR_OK;
}

void ear_comm_destroy(ear_comm_t comm) {
  if (!comm) return;
  cudaDeviceSynchronize();
  ear::release_window(comm);
  delete comm;
}

}  // extern "C"
