// C-ABI entry points of libearapsp.so (declared and documented in include/ear_apsp.h).
#include <cstdarg>
#include <cstring>
#include <vector>

#include <cstdlib>
#include <mutex>

#include "common.cuh"

namespace ear {

static thread_local char g_err[512] = "";

void set_error(const char *fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

namespace {

__global__ void k_export(int32_t n, const VDesc *desc, const int32_t *tidv, const int32_t *earv, int32_t *tid,
                         int32_t *ear, int32_t *left, int32_t *right, int32_t *offl, int32_t *offr) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const VDesc d = desc[v];
    if (tid) tid[v] = tidv[v];
    if (ear) ear[v] = earv[v];
    if (left) left[v] = d.p;
    if (right) right[v] = d.q;
    if (offl) offl[v] = d.cp;
    if (offr) offr[v] = d.cq;
  }
}

int32_t padded(const ear_plan_s *p, int32_t nranks) {
  return (int32_t)round_up(std::max<int64_t>(p->n_reduced, 1), (int64_t)TILE * nranks);
}

bool aligned16(const void *p) { return ((uintptr_t)p & 15u) == 0; }

}  // namespace
}  // namespace ear

using namespace ear;

extern "C" {

const char *ear_last_error(void) { return g_err; }

const char *ear_version(void) { return "earapsp 0.1 (sm_100a)"; }

const char *ear_status_string(ear_status_t s) {
  switch (s) {
    case EAR_OK: return "EAR_OK";
    case EAR_EINVAL: return "EAR_EINVAL";
    case EAR_ENOMEM: return "EAR_ENOMEM";
    case EAR_ECUDA: return "EAR_ECUDA";
    case EAR_ENCCL: return "EAR_ENCCL";
    case EAR_EOVERFLOW: return "EAR_EOVERFLOW";
    case EAR_EUNSUPPORTED: return "EAR_EUNSUPPORTED";
  }
  return "EAR_?";
}

void ear_row_block(int32_t rows, int32_t nranks, int32_t rank, int32_t *begin, int32_t *end) {
  if (nranks < 1) nranks = 1;
  if (begin) *begin = (int32_t)((int64_t)rows * rank / nranks);
  if (end) *end = (int32_t)((int64_t)rows * (rank + 1) / nranks);
}

}  // extern "C"

namespace {
// The library's scratch (D, piece pool, expansion buffers) comes from the device's default stream-ordered
// pool.  With its default release threshold (0) the pool hands its memory back to the driver at every
// synchronisation and the next call maps it again; keep it instead (EAR_POOL_KEEP=0 keeps the driver
// default).  Once per device, thread-safe.
void keep_pool_memory() {
  static std::once_flag once[64];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return;
  std::call_once(once[dev], [dev] {
    const char *e = getenv("EAR_POOL_KEEP");
    if (e && atoi(e) == 0) return;
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
      uint64_t keep = UINT64_MAX;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    }
    cudaGetLastError();
  });
}
}  // namespace

extern "C" {

ear_status_t ear_decompose(int32_t n, int64_t m, const int32_t *d_src, const int32_t *d_dst, const int32_t *d_w,
                           uint32_t flags, void *stream, ear_plan_t *out) {
  NvtxRange nvtx_("ear: Phase I ear_decompose");
  g_err[0] = 0;
  keep_pool_memory();
  if (!out) { set_error("ear_decompose: out is NULL"); return EAR_EINVAL; }
  *out = nullptr;
  if (n < 1 || m < 0 || (m > 0 && (!d_src || !d_dst || !d_w)) || 2 * m > (int64_t)INT32_MAX) {
    set_error("ear_decompose: bad sizes n=%d m=%lld", n, (long long)m);
    return EAR_EINVAL;
  }
  ear_plan_s *p = new ear_plan_s;
  cudaGetDevice(&p->device);
  int sp = prof_begin(PK_DECOMPOSE, (cudaStream_t)stream);
  ear_status_t s = decompose(n, m, d_src, d_dst, d_w, flags, (cudaStream_t)stream, p);
  prof_end(sp, (cudaStream_t)stream, 0);
  if (s != EAR_OK) {
    cudaStreamSynchronize((cudaStream_t)stream);
    plan_free(p);
    delete p;
    return s;
  }
  *out = p;
  return EAR_OK;
}

ear_status_t ear_plan_info(ear_plan_t p, int32_t nranks, ear_plan_info_t *info) {
  if (!p || !info || nranks < 1) { set_error("ear_plan_info: bad arguments"); return EAR_EINVAL; }
  info->n = p->n;
  info->n_reduced = p->n_reduced;
  info->n_reduced_padded = padded(p, nranks);
  info->n_chains = p->n_chains;
  info->max_chain_len = p->max_chain_len;
  info->n_promoted = p->n_promoted;
  info->n_reduced_edges = p->n_redges;
  info->m_simple = p->m_simple;
  info->rank_rounds = p->rank_rounds;
  info->max_weight = p->max_weight;
  return EAR_OK;
}

ear_status_t ear_plan_export(ear_plan_t p, int32_t *d_tid, int32_t *d_ear, int32_t *d_left, int32_t *d_right,
                             int32_t *d_off_left, int32_t *d_off_right, void *stream) {
  if (!p) { set_error("ear_plan_export: NULL plan"); return EAR_EINVAL; }
  int grid = (int)std::min<int64_t>(ceil_div(p->n, 256), 4096);
  EAR_LAUNCH(k_export, grid, 256, 0, (cudaStream_t)stream)(p->n, p->desc, p->tid, p->ear, d_tid, d_ear, d_left, d_right,
                                                    d_off_left, d_off_right);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

ear_status_t ear_plan_export_reduced_edges(ear_plan_t p, int32_t *d_u, int32_t *d_v, int32_t *d_w, void *stream) {
  if (!p) { set_error("ear_plan_export_reduced_edges: NULL plan"); return EAR_EINVAL; }
  if (p->n_redges == 0) return EAR_OK;
  cudaStream_t st = (cudaStream_t)stream;
  size_t b = sizeof(int32_t) * (size_t)p->n_redges;
  if (d_u) EAR_CUDA_TRY(cudaMemcpyAsync(d_u, p->re_u, b, cudaMemcpyDeviceToDevice, st));
  if (d_v) EAR_CUDA_TRY(cudaMemcpyAsync(d_v, p->re_v, b, cudaMemcpyDeviceToDevice, st));
  if (d_w) EAR_CUDA_TRY(cudaMemcpyAsync(d_w, p->re_w, b, cudaMemcpyDeviceToDevice, st));
  return EAR_OK;
}

void ear_plan_destroy(ear_plan_t p) {
  if (!p) return;
  plan_free(p);
  delete p;
}

ear_status_t apsp_reduced(ear_plan_t p, int32_t *d_D, int64_t ldd, ear_comm_t comm, void *stream) {
  NvtxRange nvtx_("ear: Phase II apsp_reduced");
  g_err[0] = 0;
  if (!p || !d_D) { set_error("apsp_reduced: NULL argument"); return EAR_EINVAL; }
  const int32_t P = comm ? comm->nranks : 1;
  const int32_t Np = padded(p, P);
  if (ldd < Np || ldd % 4 != 0 || !aligned16(d_D)) {
    set_error("apsp_reduced: need ldd >= Np=%d, ldd %% 4 == 0 and a 16-byte aligned D (ldd=%lld)", Np,
              (long long)ldd);
    return EAR_EINVAL;
  }
  cudaStream_t st = (cudaStream_t)stream;
  if (!comm) {
    if (p->flags & EAR_FLAG_PART) {
      bool applied = false;
      EAR_TRY(part_rows(p, nullptr, 0, d_D, ldd, Np, &applied, st));
      if (applied) return EAR_OK;
    }
    if (p->flags & EAR_FLAG_BCC) return bcc_solve(p, nullptr, d_D, ldd, Np, 0, Np, nullptr, st);
    if (p->flags & EAR_FLAG_SSSP) return sssp_rows(p, d_D, ldd, Np, 0, Np, nullptr, st);
    EAR_TRY(fw_init_D(p, d_D, ldd, Np, 0, Np, st));
    const bool allow16 = !(p->flags & EAR_FLAG_FW32);
    const int32_t *lab = nullptr;
    if (allow16) EAR_TRY(reduced_labels(p, Np, st, &lab));
    return fw_single(d_D, ldd, Np, st, lab, p->n_reduced, allow16, p);
  }
  // with a communicator -- even one of a single rank -- d_D holds this rank's owned tile rows
  // (zig-zag assignment, ascending) and the sharded schedule with its NCCL calls runs
  const int32_t nt = Np / TILE;
  int32_t *d_rows = nullptr, nown = 0;
  EAR_TRY(shard_rows_device(nt, P, comm->rank, &d_rows, &nown, st));
  ear_status_t s = EAR_OK;
  if (p->flags & EAR_FLAG_BCC) {   // largest piece sharded, owned rows composed
    s = bcc_solve(p, comm, d_D, ldd, Np, 0, nown * TILE, d_rows, st);
  } else if (p->flags & EAR_FLAG_SSSP) {   // every rank its own rows: no exchange in Phase II
    s = sssp_rows(p, d_D, ldd, Np, 0, nown * TILE, d_rows, st);
  } else {
    std::vector<int32_t> rows(nown);
    if (nown > 0) {
      Readback rb(st);
      cudaError_t e = rb.get(rows.data(), d_rows, sizeof(int32_t) * nown);
      if (e == cudaSuccess) e = rb.sync();
      if (e != cudaSuccess) { set_error("apsp_reduced: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
    }
    for (int32_t b = 0; b < nown && s == EAR_OK; ++b)
      s = fw_init_D(p, d_D + (int64_t)b * TILE * ldd, ldd, Np, rows[b] * TILE, TILE, st);
    const bool allow16 = !(p->flags & EAR_FLAG_FW32);
    const int32_t *lab = nullptr;
    if (s == EAR_OK && allow16) s = reduced_labels(p, Np, st, &lab);
    if (s == EAR_OK) s = fw_sharded_auto(d_D, ldd, Np, comm, lab, p->n_reduced, allow16, st, p);
  }
  cudaFreeAsync(d_rows, st);
  return s;
}

ear_status_t apsp_reduced_emulated(ear_plan_t p, int32_t nranks, int32_t *d_D, int64_t ldd, void *stream) {
  g_err[0] = 0;
  if (!p || !d_D || nranks < 1) { set_error("apsp_reduced_emulated: bad argument"); return EAR_EINVAL; }
  const int32_t Np = padded(p, nranks);
  if (ldd < Np || ldd % 4 != 0 || !aligned16(d_D)) {
    set_error("apsp_reduced_emulated: need ldd >= Np=%d, ldd %% 4 == 0, 16-byte aligned D", Np);
    return EAR_EINVAL;
  }
  return fw_sharded_emulated(p, d_D, ldd, Np, nranks, (cudaStream_t)stream);
}

ear_status_t apsp_reduced_rank_timing(ear_plan_t p, int32_t nranks, int32_t rank, void *stream) {
  g_err[0] = 0;
  if (!p || nranks < 1 || rank < 0 || rank >= nranks) {
    set_error("apsp_reduced_rank_timing: bad argument");
    return EAR_EINVAL;
  }
  return fw_rank_timing(p, padded(p, nranks), nranks, rank, (p->flags & EAR_FLAG_FW32) != 0, (cudaStream_t)stream);
}

int32_t ear_owned_tile_rows(int32_t n_reduced_padded, int32_t nranks, int32_t rank) {
  if (nranks < 1 || rank < 0 || rank >= nranks) return 0;
  return shard_nown(n_reduced_padded / TILE, nranks, rank);
}

ear_status_t ear_gather_reduced(ear_plan_t p, const int32_t *d_D_block, int64_t ldd_block, int32_t *d_D_full,
                                int64_t ldd_full, ear_comm_t comm, void *stream) {
  if (!p || !d_D_block || !d_D_full) { set_error("ear_gather_reduced: NULL argument"); return EAR_EINVAL; }
  cudaStream_t st = (cudaStream_t)stream;
  const int32_t P = comm ? comm->nranks : 1;
  const int32_t Np = padded(p, P);
  if (ldd_block < Np || ldd_full < Np) { set_error("ear_gather_reduced: leading dimension < Np"); return EAR_EINVAL; }
  if (!comm) {
    if (d_D_block != d_D_full)
      EAR_CUDA_TRY(cudaMemcpy2DAsync(d_D_full, sizeof(int32_t) * ldd_full, d_D_block, sizeof(int32_t) * ldd_block,
                                     sizeof(int32_t) * Np, Np, cudaMemcpyDeviceToDevice, st));
    return EAR_OK;
  }
  return fw_sharded_gather(d_D_block, ldd_block, Np, d_D_full, ldd_full, comm, st);
}

ear_status_t expand_ears(ear_plan_t p, const int32_t *d_D_full, int64_t ldd, int32_t row_begin, int32_t row_end,
                         int32_t *d_out, int64_t ldo, void *stream) {
  NvtxRange nvtx_("ear: Phase III expand_ears");
  g_err[0] = 0;
  if (!p || !d_D_full || (!d_out && row_end > row_begin)) { set_error("expand_ears: NULL argument"); return EAR_EINVAL; }
  if (row_begin < 0 || row_end < row_begin || row_end > p->n || ldo < p->n || ldd < p->n_reduced) {
    set_error("expand_ears: bad range [%d,%d) of n=%d or ldo=%lld / ldd=%lld too small", row_begin, row_end, p->n,
              (long long)ldo, (long long)ldd);
    return EAR_EINVAL;
  }
  return expand(p, d_D_full, ldd, row_begin, row_end, d_out, ldo, (cudaStream_t)stream);
}

ear_status_t ear_query_pairs(ear_plan_t p, const int32_t *d_D_full, int64_t ldd, int64_t npairs, const int32_t *d_s,
                             const int32_t *d_t, int32_t *d_out, void *stream) {
  NvtxRange nvtx_("ear: query pairs");
  g_err[0] = 0;
  if (!p || !d_D_full || npairs < 0 || (npairs > 0 && (!d_s || !d_t || !d_out)) || ldd < p->n_reduced) {
    set_error("ear_query_pairs: bad argument");
    return EAR_EINVAL;
  }
  return query_pairs(p, d_D_full, ldd, npairs, d_s, d_t, d_out, (cudaStream_t)stream);
}

// D as Phase III reads it: the int32 Np x Np matrix, or -- on the single-GPU Phase II by blocks, when
// the pair-major expansion applies and every distance fits -- only its u16 rows (half the bytes, and the
// expansion stages them without a narrowing pass)
struct DKeep {
  int32_t *D = nullptr;
  uint16_t *D16 = nullptr;
  int32_t ld16 = 0;
};

static ear_status_t expand_kept(ear_plan_s *p, const DKeep &k, int32_t Np, int32_t r0, int32_t r1, int32_t *out,
                                int64_t ldo, cudaStream_t st) {
  if (k.D16) return expand_from16(p, k.D16, k.ld16, r0, r1, out, ldo, st);
  return expand(p, k.D, Np, r0, r1, out, ldo, st);
}

static void free_kept(DKeep &k, cudaStream_t st) {
  if (k.D) cudaFreeAsync(k.D, st);
  if (k.D16) cudaFreeAsync(k.D16, st);
  k = DKeep{};
}

// Phases II + III for an existing plan into device rows (shared by apsp_full / apsp_full_host).
// `u16_ok`: the rows Phase III will write are 16-byte aligned with ldo % 4 == 0 (the pair-major kernel's
// stores).  With `keep` D is handed back (not freed) for later expansions.
static ear_status_t solve_rows(ear_plan_s *p, int32_t row_begin, int32_t row_end, int32_t *d_out, int64_t ldo,
                               ear_comm_t comm, cudaStream_t st, DKeep *keep, bool u16_ok) {
  NvtxRange nvtx_("ear: Phases II + III");
  const int32_t P = comm ? comm->nranks : 1;
  const int32_t Np = padded(p, P);
  DKeep k;
  ear_status_t s = EAR_OK;
  LabTrace tr(st, -3);
  // the expansion's item lists: when the host can predict that they apply (no device check needed),
  // they are enqueued from inside Phase II, while its last products run, so their host-side launch
  // cost overlaps GPU work instead of delaying Phase II
  bool part_xp = false;
  bool xp_done = false;
  const bool part_pred = (p->flags & EAR_FLAG_PART) && u16_ok && xp_predict(p);
  if ((p->flags & EAR_FLAG_PART) && u16_ok && !part_pred) part_xp = xp_applicable(p, st), xp_done = true;
  if (part_pred || part_xp) {
    tr.mark("solve: xp lists");
    // Phase II by regions straight into u16 rows; every rank computes all of D (a few ms) and expands
    // only its own output rows, so no exchange is needed
    k.ld16 = xp_row_stride(p);
    EAR_CUDA_TRY(cudaMallocAsync((void **)&k.D16, sizeof(uint16_t) * (size_t)p->n_reduced * k.ld16, st));
    bool applied = false;
    s = part_rows(p, k.D16, k.ld16, nullptr, 0, 0, &applied, st, row_begin, row_end, [&] {
      if (!xp_done) part_xp = xp_applicable(p, st), xp_done = true;
    });
    if (s == EAR_OK && !xp_done) part_xp = xp_applicable(p, st), xp_done = true;
    if (s != EAR_OK || !applied || !part_xp) {
      cudaFreeAsync(k.D16, st);
      k.D16 = nullptr;
    }
  }
  if (s == EAR_OK && !k.D16 && !comm && (p->flags & EAR_FLAG_BCC) && u16_ok && xp_applicable(p, st)) {
    k.ld16 = xp_row_stride(p);
    int32_t *flag = nullptr;
    EAR_CUDA_TRY(cudaMallocAsync((void **)&k.D16, sizeof(uint16_t) * (size_t)p->n_reduced * k.ld16, st));
    EAR_CUDA_TRY(cudaMallocAsync((void **)&flag, sizeof(int32_t), st));
    EAR_CUDA_TRY(dev_memset(flag, 0, sizeof(int32_t), st));
    s = bcc_solve(p, nullptr, nullptr, Np, Np, 0, p->n_reduced, nullptr, st, k.D16, k.ld16, flag);
    int32_t h_flag = 1;
    if (s == EAR_OK) {
      Readback rb(st);
      cudaError_t e = rb.get(&h_flag, flag, sizeof(int32_t));
      if (e == cudaSuccess) e = rb.sync();
      if (e != cudaSuccess) { set_error("solve_rows: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
    }
    cudaFreeAsync(flag, st);
    if (s == EAR_OK && h_flag) {   // a finite distance >= 0xFFFF: the int32 D after all
      cudaFreeAsync(k.D16, st);
      k.D16 = nullptr;
    }
  }
  if (s == EAR_OK && !k.D16 && !comm && (p->flags & EAR_FLAG_SSSP) && !(p->flags & EAR_FLAG_BCC) && u16_ok &&
      xp_applicable(p, st)) {
    // per-source SSSP straight into u16 rows: no int32 D, no narrowing pass
    k.ld16 = xp_row_stride(p);
    EAR_CUDA_TRY(cudaMallocAsync((void **)&k.D16, sizeof(uint16_t) * (size_t)p->n_reduced * k.ld16, st));
    bool applied = false;
    s = sssp_rows16(p, k.D16, k.ld16, &applied, st);
    if (s != EAR_OK || !applied) {
      cudaFreeAsync(k.D16, st);
      k.D16 = nullptr;
    }
  }
  if (s == EAR_OK && !k.D16) {
    if (!comm) {
      EAR_CUDA_TRY(cudaMallocAsync((void **)&k.D, sizeof(int32_t) * (size_t)Np * Np, st));
      s = apsp_reduced(p, k.D, Np, nullptr, st);
    } else if (p->flags & EAR_FLAG_BCC) {
      // every rank holds every solved piece after bcc_solve: compose the full matrix directly, no gather
      EAR_CUDA_TRY(cudaMallocAsync((void **)&k.D, sizeof(int32_t) * (size_t)Np * Np, st));
      s = bcc_solve(p, comm, k.D, Np, Np, 0, Np, nullptr, st);
    } else {
      // the owned rows live in this rank's exchange window, where the gather reads them
      int32_t *S = nullptr;
      EAR_CUDA_TRY(cudaMallocAsync((void **)&k.D, sizeof(int32_t) * (size_t)Np * Np, st));
      s = fw_shard_buffer(comm, Np, st, &S);
      if (s == EAR_OK) s = apsp_reduced(p, S, Np, comm, st);
      if (s == EAR_OK) s = ear_gather_reduced(p, S, Np, k.D, Np, comm, st);
    }
  }
  tr.mark("solve: phase II");
  if (s == EAR_OK && d_out) s = expand_kept(p, k, Np, row_begin, row_end, d_out, ldo, st);
  tr.mark("solve: expansion");
  if (keep && s == EAR_OK) {
    *keep = k;
  } else {
    free_kept(k, st);
  }
  return s;
}

static bool rows_aligned(const int32_t *out, int64_t ldo) {
  return (ldo & 3) == 0 && (reinterpret_cast<uintptr_t>(out) & 15) == 0;
}

ear_status_t apsp_full(int32_t n, int64_t m, const int32_t *d_src, const int32_t *d_dst, const int32_t *d_w,
                       uint32_t flags, int32_t row_begin, int32_t row_end, int32_t *d_out, int64_t ldo,
                       ear_comm_t comm, void *stream) {
  NvtxRange nvtx_("ear: apsp_full");
  cudaStream_t st = (cudaStream_t)stream;
  if (row_begin < 0 || row_end < row_begin || row_end > n || ldo < n) {
    set_error("apsp_full: bad row range [%d,%d) or ldo=%lld for n=%d", row_begin, row_end, (long long)ldo, n);
    return EAR_EINVAL;
  }
  ear_plan_t p = nullptr;
  LabTrace tr(st, -4);
  EAR_TRY(ear_decompose(n, m, d_src, d_dst, d_w, flags, stream, &p));
  tr.mark("apsp_full: decompose");
  ear_status_t s = solve_rows(p, row_begin, row_end, d_out, ldo, comm, st, nullptr, rows_aligned(d_out, ldo));
  cudaError_t e = cudaStreamSynchronize(st);
  ear_plan_destroy(p);
  if (s == EAR_OK && e != cudaSuccess) {
    set_error("apsp_full: %s", cudaGetErrorString(e));
    s = EAR_ECUDA;
  }
  return s;
}

}  // extern "C"

struct ear_job_s {
  ear_plan_s *plan = nullptr;
  DKeep D;
  int32_t *buf[2] = {nullptr, nullptr};
  cudaStream_t es = nullptr;                      // expansion stream
  cudaEvent_t ev_fw = nullptr, ready[2] = {nullptr, nullptr}, freed[2] = {nullptr, nullptr}, done = nullptr;
  ear_status_t status = EAR_OK;
};

namespace {
// the device's host-copy stream: every job's D2H copies, in issue order
cudaStream_t host_copy_stream() {
  static cudaStream_t cs[64] = {};
  static std::mutex mu;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
  std::lock_guard<std::mutex> lk(mu);
  if (!cs[dev] && cudaStreamCreateWithFlags(&cs[dev], cudaStreamNonBlocking) != cudaSuccess) cs[dev] = nullptr;
  return cs[dev];
}

void job_release(ear_job_s *j) {
  if (j->done) cudaEventSynchronize(j->done);
  // stream-ordered frees only: a cudaFree would synchronise the whole device, i.e. wait for the NEXT
  // job's Phase II too and serialise the pipeline
  cudaStream_t fs = j->es ? j->es : cudaStreamPerThread;
  free_kept(j->D, fs);
  for (int i = 0; i < 2; ++i)
    if (j->buf[i]) cudaFreeAsync(j->buf[i], fs);
  cudaStreamSynchronize(fs);
  for (int i = 0; i < 2; ++i) {
    if (j->ready[i]) cudaEventDestroy(j->ready[i]);
    if (j->freed[i]) cudaEventDestroy(j->freed[i]);
  }
  if (j->ev_fw) cudaEventDestroy(j->ev_fw);
  if (j->done) cudaEventDestroy(j->done);
  if (j->es) cudaStreamDestroy(j->es);
  if (j->plan) ear_plan_destroy(j->plan);
  delete j;
}
}  // namespace

extern "C" {

ear_status_t apsp_full_host_async(int32_t n, int64_t m, const int32_t *h_src, const int32_t *h_dst, const int32_t *h_w,
                                  uint32_t flags, int32_t row_begin, int32_t row_end, int32_t *h_out, int64_t ldo,
                                  ear_comm_t comm, void *stream, ear_job_t *job) {
  cudaStream_t st = (cudaStream_t)stream;
  if (!job || row_begin < 0 || row_end < row_begin || row_end > n || ldo < n ||
      (m > 0 && (!h_src || !h_dst || !h_w)) || (row_end > row_begin && !h_out)) {
    set_error("apsp_full_host_async: bad arguments");
    return EAR_EINVAL;
  }
  *job = nullptr;
  cudaStream_t cs = host_copy_stream();
  if (!cs) { set_error("apsp_full_host_async: no copy stream"); return EAR_ECUDA; }
  // 1. the edges: pinned host arrays are read in place by Phase I's first kernels (zero-copy over
  // PCIe); others are copied in.  A copy would queue behind the previous job's device -> host row
  // copies on the copy engines and keep this job's Phases I-II from overlapping them.
  auto mapped = [](const int32_t *h) -> const int32_t * {
    cudaPointerAttributes a{};
    if (cudaPointerGetAttributes(&a, h) != cudaSuccess) { cudaGetLastError(); return nullptr; }
    return a.type == cudaMemoryTypeHost && a.devicePointer ? static_cast<const int32_t *>(a.devicePointer) : nullptr;
  };
  const int32_t *ms = m > 0 ? mapped(h_src) : nullptr, *md = m > 0 ? mapped(h_dst) : nullptr,
                *mw = m > 0 ? mapped(h_w) : nullptr;
  int32_t *dE = nullptr;
  const int32_t *es = ms, *ed = md, *ew = mw;
  if (m > 0 && !(ms && md && mw)) {
    const size_t eb = sizeof(int32_t) * (size_t)m;
    EAR_CUDA_TRY(cudaMallocAsync((void **)&dE, 3 * eb, st));
    EAR_CUDA_TRY(cudaMemcpyAsync(dE, h_src, eb, cudaMemcpyHostToDevice, st));
    EAR_CUDA_TRY(cudaMemcpyAsync(dE + m, h_dst, eb, cudaMemcpyHostToDevice, st));
    EAR_CUDA_TRY(cudaMemcpyAsync(dE + 2 * m, h_w, eb, cudaMemcpyHostToDevice, st));
    es = dE; ed = dE + m; ew = dE + 2 * m;
  }
  ear_job_s *j = new ear_job_s;
  ear_status_t s = ear_decompose(n, m, es, ed, ew, flags, stream, &j->plan);
  if (dE) cudaFreeAsync(dE, st);
  // 2. reduced APSP on `stream`, D kept
  // the chunk buffers below are the library's (aligned) with leading dimension n
  if (s == EAR_OK) s = solve_rows(j->plan, row_begin, row_end, nullptr, ldo, comm, st, &j->D, (n & 3) == 0);
  const int32_t P = comm ? comm->nranks : 1;
  const int32_t Np = s == EAR_OK ? padded(j->plan, P) : 0;
  // 3. expansion on the job's stream, in row chunks double-buffered against the copies
  const int32_t rows = row_end - row_begin;
  cudaError_t e = cudaSuccess;
  if (s == EAR_OK) {
    e = cudaStreamCreateWithFlags(&j->es, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&j->ev_fw, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&j->done, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventRecord(j->ev_fw, st);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(j->es, j->ev_fw, 0);
    if (e != cudaSuccess) { set_error("apsp_full_host_async: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  }
  if (s == EAR_OK && rows > 0) {
    int32_t chunk = (int32_t)std::max<int64_t>(32, std::min<int64_t>(rows, (256ll << 20) / (4ll * n)));
    chunk = (int32_t)round_up(chunk, 32);
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) {
      e = cudaMallocAsync((void **)&j->buf[i], sizeof(int32_t) * (size_t)chunk * n, j->es);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&j->ready[i], cudaEventDisableTiming);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&j->freed[i], cudaEventDisableTiming);
    }
    if (e != cudaSuccess) { set_error("apsp_full_host_async: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
    int it = 0;
    for (int32_t r = row_begin; s == EAR_OK && r < row_end; r += chunk, ++it) {
      const int b = it & 1;
      const int32_t r1 = std::min(row_end, r + chunk);
      if (it >= 2) cudaStreamWaitEvent(j->es, j->freed[b], 0);
      s = expand_kept(j->plan, j->D, Np, r, r1, j->buf[b], n, j->es);
      if (s != EAR_OK) break;
      cudaEventRecord(j->ready[b], j->es);
      cudaStreamWaitEvent(cs, j->ready[b], 0);
      e = cudaMemcpy2DAsync(h_out + (int64_t)(r - row_begin) * ldo, sizeof(int32_t) * ldo, j->buf[b],
                            sizeof(int32_t) * n, sizeof(int32_t) * n, r1 - r, cudaMemcpyDeviceToHost, cs);
      if (e != cudaSuccess) { set_error("apsp_full_host D2H: %s", cudaGetErrorString(e)); s = EAR_ECUDA; break; }
      cudaEventRecord(j->freed[b], cs);
    }
  }
  if (j->done) cudaEventRecord(j->done, cs);
  if (s != EAR_OK) {
    cudaStreamSynchronize(st);
    job_release(j);
    return s;
  }
  *job = j;
  return EAR_OK;
}

ear_status_t ear_job_wait(ear_job_t j) {
  if (!j) { set_error("ear_job_wait: NULL job"); return EAR_EINVAL; }
  cudaError_t e = cudaSuccess;
  if (j->done) e = cudaEventSynchronize(j->done);
  if (e == cudaSuccess && j->es) e = cudaStreamSynchronize(j->es);
  ear_status_t s = j->status;
  if (s == EAR_OK && e != cudaSuccess) { set_error("ear_job_wait: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  job_release(j);
  return s;
}

ear_status_t apsp_full_host(int32_t n, int64_t m, const int32_t *h_src, const int32_t *h_dst, const int32_t *h_w,
                            uint32_t flags, int32_t row_begin, int32_t row_end, int32_t *h_out, int64_t ldo,
                            ear_comm_t comm, void *stream) {
  NvtxRange nvtx_("ear: apsp_full_host");
  ear_job_t j = nullptr;
  EAR_TRY(apsp_full_host_async(n, m, h_src, h_dst, h_w, flags, row_begin, row_end, h_out, ldo, comm, stream, &j));
  ear_status_t s = ear_job_wait(j);
  cudaError_t e = cudaStreamSynchronize((cudaStream_t)stream);
  if (s == EAR_OK && e != cudaSuccess) { set_error("apsp_full_host: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  return s;
}

}  // extern "C"
