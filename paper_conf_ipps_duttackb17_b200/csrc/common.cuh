// Shared internals of libearapsp.so (product path only; nothing here is shared with oracle/).
#pragma once
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <functional>
#include <vector>
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include "ear_apsp.h"

namespace ear {

constexpr int TILE = EAR_TILE;   // FW tile (B)
constexpr int32_t INF = EAR_INF;

// thread-local last-error text
void set_error(const char *fmt, ...);

#define EAR_CUDA_TRY(expr)                                                                   \
  do {                                                                                       \
    cudaError_t _e = (expr);                                                                 \
    if (_e != cudaSuccess) {                                                                 \
      ::ear::set_error("%s:%d %s: %s", __FILE__, __LINE__, #expr, cudaGetErrorString(_e));   \
      return EAR_ECUDA;                                                                      \
    }                                                                                        \
  } while (0)

#define EAR_TRY(expr)                  \
  do {                                 \
    ear_status_t _s = (expr);          \
    if (_s != EAR_OK) return _s;       \
  } while (0)

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
inline int64_t round_up(int64_t a, int64_t b) { return ceil_div(a, b) * b; }

// Per-vertex expansion descriptor (16 B): p = tid(left end), cp = along-chain distance to it,
// q = tid(right end), cq = distance to it.  Terminals: p = q = own tid, cp = cq = 0.
struct __align__(16) VDesc {
  int32_t p, cp, q, cq;
};

// up to EAR_MAX_RANKS pointers, passed to kernels by value (one per rank: peer windows, destinations)
struct PeerPtrs {
  char *p[EAR_MAX_RANKS];
  int32_t n;
};

}  // namespace ear

struct ear_bcc_s;   // bcc.cu: block structure of G^r and the piece layout (EAR_FLAG_BCC)
struct ear_xp_s;    // expand.cu: the pair-major expansion's item lists (built on first use)
struct ear_part_s;  // part.cu: the region partition of G^r (EAR_FLAG_PART, built on first use)

// Library-owned plan (Reduce(G) result), device arrays unless noted.
struct ear_plan_s {
  int32_t n = 0;
  int32_t n_reduced = 0;
  int32_t n_chains = 0;
  int32_t max_chain_len = 0;
  int32_t n_promoted = 0;
  int32_t rank_rounds = 0;
  int32_t max_weight = 0;
  int64_t m_simple = 0;
  int64_t n_redges = 0;
  uint32_t flags = 0;
  int device = 0;
  cudaStream_t stream = nullptr;   // creation stream; plan arrays are freed on it (stream order)
  // per vertex
  ear::VDesc *desc = nullptr;  // [n]
  int32_t *tid = nullptr;      // [n] terminal id or -1
  int32_t *ear = nullptr;      // [n] chain id or -1
  // same-ear patch structure: chain vertices grouped by chain, sorted by off_left
  int32_t *seg_of = nullptr;    // [n] segment (chain) index of a chain vertex, -1 for terminals
  int32_t *seg_start = nullptr; // [n_chains + 1]
  int32_t *seg_vert = nullptr;  // [#chain vertices]
  int32_t n_chain_vertices = 0;
  // reduced arcs (both directions, before the P:90 min)
  int32_t *re_u = nullptr, *re_v = nullptr, *re_w = nullptr;
  int32_t *re_x = nullptr;      // first vertex after re_u on the arc: the chain's first interior vertex, -1 if direct
  // reduced-graph CSR for the per-source SSSP Phase II (built on first use)
  int32_t *r_rowptr = nullptr, *r_col = nullptr, *r_w = nullptr;
  void *r_arcs = nullptr;       // packed (col, w) int2 arcs: ELL rows of r_ell_k per vertex, or CSR order
  int32_t r_ell_k = -1;
  uint32_t *r_ell16 = nullptr;  // u16 route: ELL rows of r_k16 packed arcs (target | min(w, 0xFFFF) << 16)
  int32_t r_k16 = -1;           // 0: the u16 route does not apply (N_r >= 0xFFFF or a degree > 16)
  uint32_t r_delta = 0;         // near-far step of the u16 SSSP (16 x the mean arc weight)
  uint16_t *r_maxnb = nullptr;  // largest neighbour id per reduced vertex (the SSSP's known-prefix boundary)
  int32_t n_rarcs = 0;
  ear_bcc_s *bcc = nullptr;     // built on first use (EAR_FLAG_BCC, ear_bcc_info)
  int32_t *cc = nullptr;        // [cc_np] connected-component labels of G^r (16-bit FW range check)
  ear_xp_s *xp = nullptr;       // pair-major expansion items (expand.cu), built on first use
  ear_part_s *part = nullptr;   // region partition (part.cu), built on first use
  int32_t connected = -1;       // G^r has one connected component: 1 / 0, -1 unknown (set with the partition)
  int32_t cc_np = 0;
};

// Library-owned communicator (comm.cu): the ranks' peer-mapped windows and the flag sequences.
struct ear_comm_s {
  int32_t nranks = 1;
  int32_t rank = 0;
  int device = 0;
  ear_allgather_fn allgather = nullptr;   // caller's host all-gather (handle exchange only)
  void *ctx = nullptr;
  char *win = nullptr;                    // this rank's window (cudaMalloc, IPC-exported)
  size_t win_bytes = 0;
  char *peer[EAR_MAX_RANKS] = {};         // every rank's window mapped here (peer[rank] == win)
  int32_t np = 0;                         // Np the window layout is cut for (comm_reserve)
  uint64_t seq_pieces = 0, seq_tile = 0, seq_barrier = 0, seq_check = 0;   // flag values, same on every rank
};

namespace ear {
// NVTX range around a phase of the path (visible in Nsight Systems / Compute timelines; header-only NVTX3,
// a few ns when no tool is attached)
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange &) = delete;
  NvtxRange &operator=(const NvtxRange &) = delete;
};
// EAR_PART_TRACE=1 (lab): host time at stage boundaries, each synchronised (stderr)
struct LabTrace {
  cudaStream_t st;
  int depth;
  bool on;
  std::chrono::steady_clock::time_point t0;
  LabTrace(cudaStream_t s, int d) : st(s), depth(d) {
    static const bool env = getenv("EAR_PART_TRACE") != nullptr;
    on = env;
    if (on) {
      cudaStreamSynchronize(st);
      t0 = std::chrono::steady_clock::now();
    }
  }
  void mark(const char *what) {
    if (!on) return;
    cudaStreamSynchronize(st);
    const auto t = std::chrono::steady_clock::now();
    fprintf(stderr, "[trace d%d] %-22s %8.3f ms\n", depth, what, std::chrono::duration<double, std::milli>(t - t0).count());
    t0 = t;
  }
};
// prof.cu
enum ProfKind { PK_DECOMPOSE, PK_FW_INIT, PK_FW_P1, PK_FW_P2, PK_FW_P3, PK_COMM, PK_EXPAND, PK_SAME_CHAIN, PK_SSSP, PK_BCC, PK_COMPOSE,
                PK_FW_P3_16, PK_FW16_CONV, PK_FW_SIDE_P1, PK_FW_SIDE_P2, PK_REREDUCE, PK_BCC_PREP, PK_EXPAND_D16,
                PK_PART, PK_PART_MP };
void prof_fw16(bool used);   // one 16-bit FW attempt: used, or fell back to int32
void count_launch(int n = 1);
int prof_begin(int kind, cudaStream_t s);                // -1 when profiling is off
void prof_end(int slot, cudaStream_t s, double work);
void prof_fw16_precheck();   // a packed FW abandoned after round 0 by its cap precheck
// Small device -> host readbacks (counts, flags, piece sizes) that bypass the copy engines: a small
// kernel stores the bytes into a slot of a mapped pinned staging buffer (1 MB per thread; a get() takes
// slots above every live object's), so a readback never queues behind a previous job's multi-GB
// device -> host row copies on the copy engine (apsp_full_host_async pipelining).  get() enqueues on the stream; sync() synchronises the stream and
// delivers every slot to its destination.  Destroyed without sync(): synchronises, delivers nothing.
class Readback {
 public:
  explicit Readback(cudaStream_t st);
  ~Readback();
  Readback(const Readback &) = delete;
  Readback &operator=(const Readback &) = delete;
  cudaError_t get(void *h_dst, const void *d_src, size_t bytes);
  cudaError_t sync();

 private:
  struct Slot { void *dst; size_t off, bytes; };
  cudaStream_t st_;
  size_t base_, used_;
  bool pending_ = false;
  std::vector<Slot> slots_;
};
// the same store straight into caller-owned pinned (mapped) host memory; completion is the caller's event
cudaError_t readback_direct(void *h_mapped, const void *d_src, size_t bytes, cudaStream_t st);
// cudaMemsetAsync / device-to-device cudaMemcpyAsync as SM kernels (prof.cu): the copy engines may be busy
// for seconds with a previous job's device -> host row copies, and an engine-side memset queues behind them
cudaError_t dev_memset(void *dst, int value, size_t bytes, cudaStream_t st);
cudaError_t dev_copy(void *dst, const void *src, size_t bytes, cudaStream_t st);
// launch one of the library's kernels and count it: EAR_LAUNCH(k, grid, block, smem, stream)(args);
#define EAR_LAUNCH(k, g, b, sm, st) ::ear::count_launch(), k<<<(g), (b), (sm), (st)>>>
// decompose.cu
ear_status_t decompose(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w,
                       uint32_t flags, cudaStream_t stream, ear_plan_s *plan);
void plan_free(ear_plan_s *plan);
// fw.cu
ear_status_t fw_init_D(const ear_plan_s *plan, int32_t *D, int64_t ldd, int32_t Np, int32_t row0,
                       int32_t rows, cudaStream_t stream);
ear_status_t fw_single(int32_t *D, int64_t ldd, int32_t Np, cudaStream_t stream, const int32_t *lab = nullptr,
                       int32_t n_real = 0, bool allow16 = false, ear_plan_s *plan = nullptr);
ear_status_t reduced_labels(ear_plan_s *p, int32_t Np, cudaStream_t st, const int32_t **out);
// row-block sharding: rank r owns the tile rows ti with (ti mod 2P) in {r, 2P-1-r} (zig-zag), stored
// ascending as 128-row blocks; the exchange runs over the communicator's peer windows (comm.cu)
std::vector<int32_t> shard_rows(int32_t nt, int32_t P, int32_t rank);
// the packed schedule first (allow16; lab / n_real as for fw_single), else the int32 one; collective
ear_status_t fw_sharded_auto(int32_t *S, int64_t ldd, int32_t Np, ear_comm_s *comm, const int32_t *lab,
                             int32_t n_real, bool allow16, cudaStream_t stream, ear_plan_s *plan = nullptr);
// every rank's owned upper tiles -> the full matrix Df on every rank (peer reads + mirror); collective
ear_status_t fw_sharded_gather(const int32_t *S, int64_t ldd, int32_t Np, int32_t *Df, int64_t ldf, ear_comm_s *comm,
                               cudaStream_t stream);
// this rank's owned-row storage inside its window (no copy at the gather); collective
ear_status_t fw_shard_buffer(ear_comm_s *comm, int32_t Np, cudaStream_t stream, int32_t **S);
ear_status_t fw_rank_timing(const ear_plan_s *plan, int32_t Np, int32_t P, int32_t rank, bool fw32, cudaStream_t stream);
ear_status_t fw_sharded_emulated(ear_plan_s *plan, int32_t *D, int64_t ldd, int32_t Np, int32_t P,
                                 cudaStream_t stream);
int32_t shard_nown(int32_t nt, int32_t P, int32_t rank);
ear_status_t shard_rows_device(int32_t nt, int32_t P, int32_t rank, int32_t **d_rows, int32_t *nown,
                               cudaStream_t stream);
// sssp.cu
// rows [row0, row0+rows) of D, or -- with d_tile_rows -- the 128-row blocks listed there (local block b
// holds global rows d_tile_rows[b]*128 ..), written consecutively into D
ear_status_t sssp_rows(ear_plan_s *plan, int32_t *D, int64_t ldd, int32_t Np, int32_t row0, int32_t rows,
                       const int32_t *d_tile_rows, cudaStream_t stream);
// every row of D (reduced vertex order, 0xFFFF = INF, stride ld16 >= round_up(N_r, 8)) by the u16 SSSP;
// *applied = false when the route does not apply or a finite distance >= 0xFFFF exists (D16 unusable)
ear_status_t sssp_rows16(ear_plan_s *plan, uint16_t *D16, int64_t ld16, bool *applied, cudaStream_t stream);
// bcc.cu -- Phase II by biconnected pieces (paper sec. 2.2)
ear_status_t bcc_prepare(ear_plan_s *plan, int32_t P, cudaStream_t stream);
// D16 / ld16 / flag16 (optional): also (or, with D == NULL, only) the rows as u16 for the pair-major
// expansion (0xFFFF = INF); *flag16 set when a finite distance does not fit (then D16 is unusable)
ear_status_t bcc_solve(ear_plan_s *plan, ear_comm_s *comm, int32_t *D, int64_t ldd, int32_t Np, int32_t row0,
                       int32_t rows, const int32_t *d_tile_rows, cudaStream_t stream, uint16_t *D16 = nullptr,
                       int64_t ld16 = 0, int32_t *flag16 = nullptr);
void bcc_free(ear_bcc_s *b, cudaStream_t stream);
// part.cu -- Phase II by regions (EAR_FLAG_PART): every row of D as u16 into D16 (ld16 >= round_up(N_r, 8)),
// or (D16 == NULL) widened into the int32 Np x Np matrix D; *applied = false when the route does not apply
ear_status_t part_prepare(ear_plan_s *plan, cudaStream_t stream);
// row_begin / row_end (D16 only): the caller's rows of G; D16 then holds only the rows Phase III stages
// for them (the regions of their chain ends)
// before_sync (optional): called once the last products are enqueued, before the final readback (host
// work to overlap with them)
ear_status_t part_rows(ear_plan_s *plan, uint16_t *D16, int64_t ld16, int32_t *D, int64_t ldd, int32_t Np,
                       bool *applied, cudaStream_t stream, int32_t row_begin = 0, int32_t row_end = 0,
                       const std::function<void()> &before_sync = nullptr);
void part_free(ear_part_s *q, cudaStream_t stream);
// expand.cu
ear_status_t expand(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t row_begin,
                    int32_t row_end, int32_t *out, int64_t ldo, cudaStream_t stream, int prof_kind = PK_EXPAND);
// the pair-major expansion straight from u16 rows of D (0xFFFF = INF, row stride ld16 = xp_row_stride):
// the path apsp_full takes when Phase II can hand over D16 (bcc_solve's u16 output)
int32_t xp_row_stride(const ear_plan_s *plan);
bool xp_applicable(ear_plan_s *plan, cudaStream_t stream);   // builds the item lists on first use
bool xp_bounds_fit(const ear_plan_s *plan);
bool xp_predict(const ear_plan_s *plan);   // xp_applicable's answer, known without building the lists
ear_status_t expand_from16(const ear_plan_s *plan, const uint16_t *D16, int32_t ld16, int32_t row_begin,
                           int32_t row_end, int32_t *out, int64_t ldo, cudaStream_t stream, int prof_kind = PK_EXPAND);
void xp_free(ear_xp_s *xp, cudaStream_t stream);
ear_status_t query_pairs(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int64_t npairs, const int32_t *qs,
                         const int32_t *qt, int32_t *out, cudaStream_t stream);
// comm.cu -- peer-memory transport (window layout in comm.cu)
enum { SLOT_PIECES = 0, SLOT_TILE = 64, SLOT_BARRIER = 128, SLOT_CHECK = 192 };
size_t comm_win_bytes(int32_t Np, int32_t nown);
ear_status_t comm_reserve(ear_comm_s *c, int32_t Np, int32_t nown, cudaStream_t st);   // collective
char *comm_L(ear_comm_s *c, int p, int b);          // rank p's L[b] as mapped here
char *comm_stage(ear_comm_s *c, int p, int b);      // rank p's stage[b]
int32_t *comm_region(ear_comm_s *c, int p);         // rank p's owned-rows region
PeerPtrs comm_flags_all(ear_comm_s *c);             // every rank's window base (flag slots at offset 0)
ear_status_t comm_signal(ear_comm_s *c, int32_t slot, uint64_t value, cudaStream_t st);
ear_status_t comm_wait(ear_comm_s *c, int32_t slot, uint64_t value, cudaStream_t st);
ear_status_t comm_wait_one(ear_comm_s *c, int32_t slot, uint64_t value, cudaStream_t st);
ear_status_t comm_barrier(ear_comm_s *c, cudaStream_t st);
// helpers (prof.cu): per-device SM count; cudaFuncSetAttribute(max dynamic smem) once
// per (device, kernel), thread-safe
int num_sms();
cudaError_t smem_attr(const void *kernel, int bytes);
}  // namespace ear
