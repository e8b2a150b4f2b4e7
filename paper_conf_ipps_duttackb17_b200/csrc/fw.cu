// Phase II -- S^r = APSP(G^r) (Alg. 1 lines 4-7) as a three-phase blocked min-plus
// Floyd-Warshall (blocked FW of [23], cited at P:60) over 128 x 128 int32 tiles on sm_100a.
//
//   D init   INF everywhere, 0 on the diagonal, atomicMin of the G^r arcs (keep the shortest of
//            parallel edges).
//   round k  phase 1  closure of the pivot tile (k,k): serial kk loop in one CTA; the matrix is
//                     symmetric (undirected G), so row kk doubles as column kk and one smem row
//                     buffer (double-buffered) broadcasts the pivot each step;
//            phase 2  pivot-row tiles (k,j): C = min(C, P (x) C) with the CLOSED pivot P -- a single
//                     min-plus product, no serial dependency (closure argument in DESIGN.md);
//            phase 3  remaining tiles (i,j): C = min(C, D[i,K] (x) D[K,j]).
//   Both phase 2 and 3 run the same register-blocked min-plus tile kernel: 256 threads, 8x8 int32
//   accumulators per thread, operands streamed through double-buffered shared memory by cp.async in
//   32-deep k-chunks; one VIADDMNMX (c = min(c, a + b)) per min-plus.  Because D is symmetric,
//   D[i,K] = D[K,i]^T: both operands are slices of the pivot ROW block, which is also the only
//   block a multi-GPU round has to broadcast.  On one GPU only the upper triangle of tiles is
//   computed and each result is written twice (tile and transposed mirror): half the min-plus work.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <vector>

#include "common.cuh"

namespace ear {
namespace {

constexpr int NT = 256;

__global__ void k_init_D(int32_t *D, int64_t ldd, int32_t Np, int32_t row0, int32_t rows) {
  int64_t total = (int64_t)rows * (Np / 4);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int32_t r = (int32_t)(i / (Np / 4));
    int32_t c4 = (int32_t)(i % (Np / 4)) * 4;
    int4 v = make_int4(INF, INF, INF, INF);
    int32_t g = row0 + r;   // global row
    if (g >= c4 && g < c4 + 4) ((int32_t *)&v)[g - c4] = 0;
    *reinterpret_cast<int4 *>(D + (int64_t)r * ldd + c4) = v;
  }
}

__global__ void k_init_edges(const int32_t *ru, const int32_t *rv, const int32_t *rw, int64_t E, int32_t *D,
                             int64_t ldd, int32_t row0, int32_t rows) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < E; i += (int64_t)gridDim.x * blockDim.x) {
    int32_t u = ru[i] - row0;
    if (u >= 0 && u < rows) atomicMin(D + (int64_t)u * ldd + rv[i], rw[i]);
  }
}

__device__ __forceinline__ int32_t mp(int32_t a, int32_t b, int32_t c) { return __viaddmin_s32(a, b, c); }

// ------------------------------------------------------------------------------ phase 1
// Closure of the 128x128 pivot tile at T (leading dimension ldt), in place.
__global__ void __launch_bounds__(NT, 1) k_fw_phase1(int32_t *T, int64_t ldt) {
  __shared__ __align__(16) int32_t rowbuf[2][TILE];
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  int32_t c[8][8];
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    const int i = (r < 4 ? 0 : 64) + ty * 4 + (r & 3);
    const int4 lo = *reinterpret_cast<const int4 *>(T + (int64_t)i * ldt + tx * 4);
    const int4 hi = *reinterpret_cast<const int4 *>(T + (int64_t)i * ldt + 64 + tx * 4);
    c[r][0] = lo.x; c[r][1] = lo.y; c[r][2] = lo.z; c[r][3] = lo.w;
    c[r][4] = hi.x; c[r][5] = hi.y; c[r][6] = hi.z; c[r][7] = hi.w;
  }
  // row 0 is owned by ty = 0, r = 0
  if (ty == 0) {
    *reinterpret_cast<int4 *>(&rowbuf[0][tx * 4]) = make_int4(c[0][0], c[0][1], c[0][2], c[0][3]);
    *reinterpret_cast<int4 *>(&rowbuf[0][64 + tx * 4]) = make_int4(c[0][4], c[0][5], c[0][6], c[0][7]);
  }
  __syncthreads();
  for (int kk = 0; kk < TILE; ++kk) {
    const int32_t *rb = rowbuf[kk & 1];
    const int4 alo = *reinterpret_cast<const int4 *>(rb + ty * 4);
    const int4 ahi = *reinterpret_cast<const int4 *>(rb + 64 + ty * 4);
    const int4 blo = *reinterpret_cast<const int4 *>(rb + tx * 4);
    const int4 bhi = *reinterpret_cast<const int4 *>(rb + 64 + tx * 4);
    const int32_t a[8] = {alo.x, alo.y, alo.z, alo.w, ahi.x, ahi.y, ahi.z, ahi.w};
    const int32_t b[8] = {blo.x, blo.y, blo.z, blo.w, bhi.x, bhi.y, bhi.z, bhi.w};
#pragma unroll
    for (int r = 0; r < 8; ++r)
#pragma unroll
      for (int q = 0; q < 8; ++q) c[r][q] = mp(a[r], b[q], c[r][q]);
    // publish row kk+1 (after this step's update) for the next step
    const int nk = kk + 1;
    if (nk < TILE && ty == ((nk & 63) >> 2)) {
      const int rr = (nk & 3) + (nk >= 64 ? 4 : 0);
      int32_t *wb = rowbuf[nk & 1];
#pragma unroll
      for (int r = 0; r < 8; ++r) {
        if (r == rr) {
          *reinterpret_cast<int4 *>(wb + tx * 4) = make_int4(c[r][0], c[r][1], c[r][2], c[r][3]);
          *reinterpret_cast<int4 *>(wb + 64 + tx * 4) = make_int4(c[r][4], c[r][5], c[r][6], c[r][7]);
        }
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    const int i = (r < 4 ? 0 : 64) + ty * 4 + (r & 3);
    *reinterpret_cast<int4 *>(T + (int64_t)i * ldt + tx * 4) = make_int4(c[r][0], c[r][1], c[r][2], c[r][3]);
    *reinterpret_cast<int4 *>(T + (int64_t)i * ldt + 64 + tx * 4) = make_int4(c[r][4], c[r][5], c[r][6], c[r][7]);
  }
}

// ------------------------------------------------------------------------------ phases 2 and 3
// Persistent, TMA-fed min-plus tile kernel.  Each CTA walks its tiles (blockIdx.x, +gridDim.x, ...);
// the operand chunks (A^T = P[k-rows][ti cols], B = P[k-rows][tj cols], 32 x 128 int32 each) stream
// through a STAGES-deep shared-memory ring filled by cp.async.bulk.tensor (TMA) and guarded by
// mbarriers (full: TMA bytes landed; empty: all 8 warps done reading), so no CTA-wide barrier sits
// in the main loop and the next tile's first chunks are fetched while the current tile finishes.
// Thread 0 doubles as the TMA producer.  The C tile lives in registers (8x8 per thread).
// MODE_CROSS / MODE_REST (single-GPU lookahead, round k): the upper tiles of row/column k+1 (without
// column k), and all upper tiles outside rows/columns k and k+1; together they are MODE_UPPER.
// MODE_LIST_CROSS / MODE_LIST_REST: the same split of a rank's MODE_LIST tiles (sharded lookahead).
// MODE_PIECES: phase 2 on the pivot-row pieces a rank contributes (owner-side phase 2, sharded FW):
// tiles (k, orow[i]) for the mk owned rows above k, then (k, k+1 ..) when the rank owns row k (posk).
enum { MODE_PIVOT_ROW = 0, MODE_UPPER = 1, MODE_LIST = 2, MODE_CROSS = 3, MODE_REST = 4, MODE_LIST_CROSS = 5,
       MODE_LIST_REST = 6, MODE_PIECES = 7 };

// Tile-kernel configuration: k-chunk depth, TMA ring depth, CTAs per SM, kk-loop unroll.
template <int KC_, int ST_, int MINB_, int UNR_>
struct FwCfg {
  static constexpr int KC = KC_;
  static constexpr int NCHUNK = TILE / KC_;
  static constexpr int SM_CHUNK = KC_ * TILE;          // ints per operand chunk
  static constexpr int STAGES = ST_;
  static constexpr int MINB = MINB_;
  static constexpr int UNR = UNR_;
  static constexpr int SMEM = STAGES * 2 * SM_CHUNK * 4 + 2 * STAGES * 8;
};

struct TileJob {
  int32_t *C;        // matrix holding the C tiles (local rows), leading dimension ldc
  int64_t ldc;
  int32_t p_row0;    // row coordinate of the pivot row block inside the operand tensor map
  int32_t k;         // pivot tile index
  int32_t nt;        // tiles per dimension (Np / 128)
  int32_t ti0;       // first local tile row (global index) of C
  int32_t nti;       // number of local tile rows
  int32_t mode;
  int32_t mirror;    // also write the transposed result into tile (tj, ti) (single GPU)
  int64_t ntiles;    // tiles in this launch
  // MODE_LIST (row-block sharded): the rank's owned tile rows (ascending), the static prefix sums of
  // their upper-tile counts (nt - ti), and per round k: mk = #owned rows < k, posk = position of row k
  // in the owned list or -1
  const int32_t *orow;
  const int64_t *opre;
  int32_t nown, mk, posk;
  int32_t posk1;     // MODE_LIST_CROSS / _REST: position of row k+1 in the owned list or -1
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
  asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n\t}\n" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t *b, uint32_t bytes) {
  asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n\t}\n" ::"r"(smem_u32(b)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try(uint64_t *b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
      : "=r"(ok)
      : "r"(smem_u32(b)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  while (!mbar_try(b, parity)) {
  }
}
// non-suspending poll (test_wait): the warp stays resident and issuing while it waits
__device__ __forceinline__ bool mbar_test(uint64_t *b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
      : "=r"(ok)
      : "r"(smem_u32(b)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait_spin(uint64_t *b, uint32_t parity) {
  while (!mbar_test(b, parity)) {
  }
}
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, int32_t c0, int32_t c1, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void tma_load_2d_hint(void *dst, const CUtensorMap *map, int32_t c0, int32_t c1, uint64_t *bar,
                                                 uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, %3}], [%4], %5;\n" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}

// decode the tile index into (ti, tj) and the local tile row lr of C
__device__ __forceinline__ void decode_tile(const TileJob &J, int64_t idx, int &ti, int &tj, int &lr) {
  const int k = J.k;
  if (J.mode == MODE_PIVOT_ROW) {
    ti = k;
    tj = (int)idx < k ? (int)idx : (int)idx + 1;
    lr = ti - J.ti0;
    return;
  }
  if (J.mode == MODE_CROSS) {
    const int j = (int)idx < k ? (int)idx : (int)idx + 1;
    ti = min(j, k + 1);
    tj = max(j, k + 1);
    lr = ti - J.ti0;
    return;
  }
  if (J.mode == MODE_UPPER || J.mode == MODE_REST) {
    // upper triangle (a <= b) of the (nt-s) x (nt-s) tiles outside the s skipped rows/columns
    // (s = 1: k; s = 2: k and k+1), row-major; row a starts at a*T - a*(a-1)/2
    const int skip = J.mode == MODE_REST ? 2 : 1;
    const int64_t T = J.nt - skip;
    double tt = (double)(2 * T + 1);
    int64_t a = (int64_t)floor((tt - sqrt(tt * tt - 8.0 * (double)idx)) * 0.5);
    if (a < 0) a = 0;
    while (a > 0 && a * T - a * (a - 1) / 2 > idx) --a;
    while ((a + 1) * T - (a + 1) * a / 2 <= idx) ++a;
    const int64_t b = a + (idx - (a * T - a * (a - 1) / 2));
    ti = (int)a < k ? (int)a : (int)a + skip;
    tj = (int)b < k ? (int)b : (int)b + skip;
    lr = ti - J.ti0;
    return;
  }
  if (J.mode == MODE_PIECES) {   // C: the rank's pieces of the pivot row block (lr 0)
    ti = k;
    tj = (int)idx < J.mk ? J.orow[idx] : k + 1 + ((int)idx - J.mk);
    lr = 0;
    return;
  }
  if (J.mode == MODE_LIST_CROSS) {   // row k+1's tiles (if owned), then tile (ti, k+1) of owned rows ti < k
    const int k1 = k + 1;
    const int nrow = J.posk1 >= 0 ? J.nt - k1 : 0;
    if ((int)idx < nrow) {
      lr = J.posk1; ti = k1; tj = k1 + (int)idx;
    } else {
      lr = (int)idx - nrow; ti = J.orow[lr]; tj = k1;
    }
    return;
  }
  // MODE_LIST: the upper tiles (ti, tj >= ti) of the owned rows, without row k and column k.
  // Per round, owned rows ti < k lose tile (ti, k) and row k (if owned) loses all its tiles.
  // MODE_LIST_REST also drops row and column k+1 (owned rows ti < k lose two tiles).
  const bool rest = J.mode == MODE_LIST_REST;
  auto pre = [&](int r) -> int64_t {
    int64_t v = J.opre[r] - (rest ? 2 : 1) * min(r, J.mk) - ((J.posk >= 0 && r > J.posk) ? (int64_t)(J.nt - k) : 0);
    if (rest && J.posk1 >= 0 && r > J.posk1) v -= J.nt - k - 1;
    return v;
  };
  int lo = 0, hi = J.nown - 1;   // largest r with pre(r) <= idx (ties: the last, skipping empty rows)
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (pre(mid) <= idx) lo = mid; else hi = mid - 1;
  }
  lr = lo;
  ti = J.orow[lo];
  tj = ti + (int)(idx - pre(lo));
  if (ti < k && tj >= k) tj += rest ? 2 : 1;
}

template <class CF>
__global__ void __launch_bounds__(NT, CF::MINB) k_fw_tiles(const __grid_constant__ CUtensorMap tmP, const TileJob J) {
  constexpr int KC = CF::KC, NCHUNK = CF::NCHUNK, SM_CHUNK = CF::SM_CHUNK, STAGES = CF::STAGES;
  extern __shared__ __align__(128) int32_t smem[];
  int32_t *sA = smem;                                   // [STAGES][KC][TILE]  A^T chunks
  int32_t *sB = sA + STAGES * SM_CHUNK;                 // [STAGES][KC][TILE]  B chunks
  uint64_t *full = reinterpret_cast<uint64_t *>(sB + STAGES * SM_CHUNK);
  uint64_t *empty = full + STAGES;
  const int tid = threadIdx.x, lane = tid & 31;
  const int tx = tid & 15, ty = tid >> 4;

  const int my_tiles = J.ntiles > (int64_t)blockIdx.x ? (int)((J.ntiles - 1 - blockIdx.x) / gridDim.x + 1) : 0;
  const int total_chunks = my_tiles * NCHUNK;
  int issued = 0;   // producer state (thread 0 only)
  auto tile_of = [&](int it, int &ti, int &tj, int &lr) {
    decode_tile(J, blockIdx.x + (int64_t)it * gridDim.x, ti, tj, lr);
  };
  auto produce = [&](int upto) {
    while (issued < upto) {
      const int st = issued % STAGES;
      if (issued >= STAGES) mbar_wait(&empty[st], (uint32_t)((issued / STAGES - 1) & 1));
      int pti, ptj, plr;
      tile_of(issued / NCHUNK, pti, ptj, plr);
      const int row = J.p_row0 + (issued % NCHUNK) * KC;
      mbar_arrive_tx(&full[st], 2 * SM_CHUNK * 4);
      tma_load_2d(sA + st * SM_CHUNK, &tmP, pti * TILE, row, &full[st]);
      tma_load_2d(sB + st * SM_CHUNK, &tmP, ptj * TILE, row, &full[st]);
      ++issued;
    }
  };

  if (tid == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], NT / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&tmP)) : "memory");
  }
  __syncthreads();
  if (tid == 0 && my_tiles > 0) produce(total_chunks < STAGES ? total_chunks : STAGES);

  int g = 0;   // chunk counter (all threads)
  for (int it = 0; it < my_tiles; ++it) {
    int ti, tj, lr;
    tile_of(it, ti, tj, lr);
    int32_t c[8][8];
    // C tile straight from global memory into registers (its latency overlaps the in-flight TMA chunks)
    int32_t *Ct = J.C + (int64_t)lr * TILE * J.ldc + (int64_t)tj * TILE;
#pragma unroll
    for (int r = 0; r < 8; ++r) {
      const int i = (r < 4 ? 0 : 64) + ty * 4 + (r & 3);
      const int4 lo = *reinterpret_cast<const int4 *>(Ct + (int64_t)i * J.ldc + tx * 4);
      const int4 hi = *reinterpret_cast<const int4 *>(Ct + (int64_t)i * J.ldc + 64 + tx * 4);
      c[r][0] = lo.x; c[r][1] = lo.y; c[r][2] = lo.z; c[r][3] = lo.w;
      c[r][4] = hi.x; c[r][5] = hi.y; c[r][6] = hi.z; c[r][7] = hi.w;
    }
#pragma unroll 1
    for (int kc = 0; kc < NCHUNK; ++kc, ++g) {
      if (tid == 0) produce(g + STAGES < total_chunks ? g + STAGES : total_chunks);
      const int st = g % STAGES;
      mbar_wait(&full[st], (uint32_t)((g / STAGES) & 1));
      const int32_t *a_s = sA + st * SM_CHUNK;
      const int32_t *b_s = sB + st * SM_CHUNK;
#pragma unroll CF::UNR
      for (int kk = 0; kk < KC; ++kk) {
        const int4 alo = *reinterpret_cast<const int4 *>(a_s + kk * TILE + ty * 4);
        const int4 ahi = *reinterpret_cast<const int4 *>(a_s + kk * TILE + 64 + ty * 4);
        const int4 blo = *reinterpret_cast<const int4 *>(b_s + kk * TILE + tx * 4);
        const int4 bhi = *reinterpret_cast<const int4 *>(b_s + kk * TILE + 64 + tx * 4);
        const int32_t a[8] = {alo.x, alo.y, alo.z, alo.w, ahi.x, ahi.y, ahi.z, ahi.w};
        const int32_t b[8] = {blo.x, blo.y, blo.z, blo.w, bhi.x, bhi.y, bhi.z, bhi.w};
#pragma unroll
        for (int r = 0; r < 8; ++r)
#pragma unroll
          for (int q = 0; q < 8; ++q) c[r][q] = mp(a[r], b[q], c[r][q]);
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[st]);
    }
    // epilogue: tile, and (single GPU, off-diagonal) its transposed mirror
#pragma unroll
    for (int r = 0; r < 8; ++r) {
      const int i = (r < 4 ? 0 : 64) + ty * 4 + (r & 3);
      *reinterpret_cast<int4 *>(Ct + (int64_t)i * J.ldc + tx * 4) = make_int4(c[r][0], c[r][1], c[r][2], c[r][3]);
      *reinterpret_cast<int4 *>(Ct + (int64_t)i * J.ldc + 64 + tx * 4) = make_int4(c[r][4], c[r][5], c[r][6], c[r][7]);
    }
    if (J.mirror && ti != tj) {
      int32_t *Mt = J.C + (int64_t)tj * TILE * J.ldc + (int64_t)ti * TILE;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const int j = (q < 4 ? 0 : 64) + tx * 4 + (q & 3);
        *reinterpret_cast<int4 *>(Mt + (int64_t)j * J.ldc + ty * 4) = make_int4(c[0][q], c[1][q], c[2][q], c[3][q]);
        *reinterpret_cast<int4 *>(Mt + (int64_t)j * J.ldc + 64 + ty * 4) = make_int4(c[4][q], c[5][q], c[6][q], c[7][q]);
      }
    }
  }
}

__global__ void k_fill(int32_t *p, int64_t n, int32_t v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}

__global__ void k_fill16(uint16_t *p, int64_t n2, uint32_t v2) {   // n2 u16 pairs
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n2; i += (int64_t)gridDim.x * blockDim.x)
    reinterpret_cast<uint32_t *>(p)[i] = v2;
}

// u16 block -> int32 (the values are capped 16-bit distances, C16 included), n % 4 == 0
__global__ void k_widen16(const uint16_t *__restrict__ P16, int32_t *__restrict__ P32, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n / 4; i += (int64_t)gridDim.x * blockDim.x) {
    const uint2 v = reinterpret_cast<const uint2 *>(P16)[i];
    reinterpret_cast<int4 *>(P32)[i] = make_int4(v.x & 0xFFFF, v.x >> 16, v.y & 0xFFFF, v.y >> 16);
  }
}

// Pivot-row block <-> a rank's owned storage, round k (prow: 128 x Np, leading dimension Np).
//   dir = 0 (gather):  prow[:, ti-block] = S(ti, k)^T for owned ti < k; prow[:, j >= k] = S(k, j) if row k owned
//   dir = 1 (scatter): the inverse, after phases 1 and 2 updated prow
// Only the pieces are launched: grid (16 sub-blocks of 32 x 32, npieces), 256 threads, where pieces
// [0, nrow) are the tiles j = k + y of the pivot row when this rank owns it (nrow = nt - k, local row
// posk) and the next mk are the owned rows ti < k (the first mk owned rows: ascending), tile (ti, k).
// TS / TP: storage / block element types (int32 <-> int32; u16 -> int32 to assemble the packed
// schedule's exchange block, u16 -> u16 to scatter its narrowed block back).
template <class TS, class TP>
__global__ void k_prow_xfer(TS *S, int64_t ldd, const int32_t *orow, int32_t k, int32_t nt, int32_t posk, TP *prow,
                            int32_t Np, int dir) {
  __shared__ uint32_t t[32][33];
  const int nrow = posk >= 0 ? nt - k : 0;
  const int y = blockIdx.y;
  const int bx = blockIdx.x & 3, by = blockIdx.x >> 2;         // 32 x 32 sub-block (bx: x, by: y)
  const int lx = threadIdx.x & 31, ly = threadIdx.x >> 5;      // 32 x 8 threads
  if (y < nrow) {              // the pivot row's upper part: plain copy, tiles j >= k
    const int lr = posk, tj = k + y;
    for (int yy = ly; yy < 32; yy += 8) {
      const int64_t row = by * 32 + yy, col = (int64_t)tj * TILE + bx * 32 + lx;
      TS *sp = S + ((int64_t)lr * TILE + row) * ldd + col;
      TP *pp = prow + row * Np + col;
      if (dir == 0) *pp = (TP)*sp; else *sp = (TS)*pp;
    }
    return;
  }
  const int lr = y - nrow, ti = orow[lr];   // owned row below the pivot: tile (ti, k) <-> prow[:, ti-block]^T
  if (dir == 0) {
    for (int yy = ly; yy < 32; yy += 8)   // S rows ti-block (bx*32+yy), cols k-block (by*32+lx)
      t[yy][lx] = (uint32_t)S[((int64_t)lr * TILE + bx * 32 + yy) * ldd + (int64_t)k * TILE + by * 32 + lx];
    __syncthreads();
    for (int yy = ly; yy < 32; yy += 8)   // prow rows (by*32+yy), cols ti-block (bx*32+lx)
      prow[(int64_t)(by * 32 + yy) * Np + (int64_t)ti * TILE + bx * 32 + lx] = (TP)t[lx][yy];
  } else {
    for (int yy = ly; yy < 32; yy += 8)
      t[yy][lx] = (uint32_t)prow[(int64_t)(by * 32 + yy) * Np + (int64_t)ti * TILE + bx * 32 + lx];
    __syncthreads();
    for (int yy = ly; yy < 32; yy += 8)
      S[((int64_t)lr * TILE + bx * 32 + yy) * ldd + (int64_t)k * TILE + by * 32 + lx] = (TS)t[lx][yy];
  }
}

// owned upper tiles (ti, tj >= ti) -> full D, and their transposed mirrors (tj, ti)
// grid: (16 sub-blocks, nt column tiles, nown owned rows), 256 threads
__global__ void k_scatter_upper(const int32_t *S, int64_t ldd, const int32_t *orow, int32_t *Df, int64_t ldf) {
  __shared__ int32_t t[32][33];
  const int lr = blockIdx.z, ti = orow[lr], tj = blockIdx.y;
  if (tj < ti) return;
  const int bx = blockIdx.x & 3, by = blockIdx.x >> 2;
  const int lx = threadIdx.x & 31, ly = threadIdx.x >> 5;
  for (int yy = ly; yy < 32; yy += 8) {
    const int32_t v = S[((int64_t)lr * TILE + by * 32 + yy) * ldd + (int64_t)tj * TILE + bx * 32 + lx];
    Df[((int64_t)ti * TILE + by * 32 + yy) * ldf + (int64_t)tj * TILE + bx * 32 + lx] = v;
    t[yy][lx] = v;
  }
  if (tj == ti) return;
  __syncthreads();
  for (int yy = ly; yy < 32; yy += 8)
    Df[((int64_t)tj * TILE + bx * 32 + yy) * ldf + (int64_t)ti * TILE + by * 32 + lx] = t[lx][yy];
}

// ------------------------------------------------------------------------------ 16-bit path
// Packed unsigned 16-bit FW (VIADDMNMX.U16x2: two min-plus per instruction, twice the int32 issue
// rate; microbench/minplus_peak.cu).  Values are capped at C16 = 0x7FFF: with a, b <= C16 the
// 16-bit sum a + b <= 0xFFFE never wraps, and FW over capped values yields exactly min(d, C16) for
// every pair (min(min(a,C)+min(b,C), C) = min(a+b, C) for a, b >= 0, so the cap commutes with every
// relaxation).  Hence every entry < C16 is the exact distance; an entry == C16 is exact (unreachable)
// iff its two vertices lie in different components -- checked afterwards, with a fall back to the
// int32 FW on the untouched int32 D when some connected pair reached the cap.
constexpr uint32_t C16 = 0x7FFF;

__global__ void k_to16(const int32_t *__restrict__ D, int64_t ldd, uint16_t *__restrict__ D16, int32_t Np) {
  const int64_t total = (int64_t)Np * (Np / 4);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / (Np / 4)), c4 = (int32_t)(i % (Np / 4)) * 4;
    const int4 v = *reinterpret_cast<const int4 *>(D + (int64_t)r * ldd + c4);
    const uint32_t lo = (uint32_t)min(v.x, (int32_t)C16) | ((uint32_t)min(v.y, (int32_t)C16) << 16);
    const uint32_t hi = (uint32_t)min(v.z, (int32_t)C16) | ((uint32_t)min(v.w, (int32_t)C16) << 16);
    *reinterpret_cast<uint2 *>(D16 + (int64_t)r * Np + c4) = make_uint2(lo, hi);
  }
}

// capped entries of connected pairs (lab[i] == lab[j]; only vertices < n_real, labels may be null:
// then [0, n_real) is one component) -> *bad
__global__ void k_check16(const uint16_t *__restrict__ D16, int32_t Np, const int32_t *__restrict__ lab, int32_t n_real,
                          int32_t *bad) {
  const int64_t total = (int64_t)Np * (Np / 8);
  int found = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / (Np / 8)), c8 = (int32_t)(i % (Np / 8)) * 8;
    if (r >= n_real || c8 >= n_real) continue;
    const uint4 v = *reinterpret_cast<const uint4 *>(D16 + (int64_t)r * Np + c8);
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const uint32_t x = (w[k >> 1] >> ((k & 1) * 16)) & 0xFFFFu;
      const int32_t c = c8 + k;
      if (x == C16 && c < n_real && (!lab || lab[r] == lab[c])) found = 1;
    }
  }
  if (__syncthreads_or(found) && threadIdx.x == 0) atomicOr(bad, 1);
}

// largest finite entry of a distance row (the cap precheck of fw_single16)
__global__ void k_row_far(const int32_t *__restrict__ row, int32_t n, int32_t *far) {
  int32_t m = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = row[i];
    if (v < INF) m = max(m, v);
  }
  m = __reduce_max_sync(0xFFFFFFFFu, m);
  if ((threadIdx.x & 31) == 0) atomicMax(far, m);
}

__global__ void k_from16(const uint16_t *__restrict__ D16, int32_t Np, int32_t *__restrict__ D, int64_t ldd) {
  const int64_t total = (int64_t)Np * (Np / 4);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / (Np / 4)), c4 = (int32_t)(i % (Np / 4)) * 4;
    const uint2 v = *reinterpret_cast<const uint2 *>(D16 + (int64_t)r * Np + c4);
    auto f = [](uint32_t x) { return x == C16 ? INF : (int32_t)x; };
    *reinterpret_cast<int4 *>(D + (int64_t)r * ldd + c4) =
        make_int4(f(v.x & 0xFFFFu), f(v.x >> 16), f(v.y & 0xFFFFu), f(v.y >> 16));
  }
}

// Pd[r][c] = P16[r][c] duplicated into both halves (the B operand of the packed product)
__global__ void k_dup16(const uint16_t *__restrict__ P16, int32_t Np, uint32_t *__restrict__ Pd) {
  const int64_t total = (int64_t)TILE * (Np / 4);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const uint2 v = reinterpret_cast<const uint2 *>(P16)[i];
    reinterpret_cast<uint4 *>(Pd)[i] = make_uint4((v.x & 0xFFFFu) * 0x10001u, (v.x >> 16) * 0x10001u,
                                                  (v.y & 0xFFFFu) * 0x10001u, (v.y >> 16) * 0x10001u);
  }
}

// ---- 16-bit row-block sharding (fw_sharded16 below)
// rows x cols block of int32 (ld lds) -> capped u16 (ld ld16); cols % 4 == 0
__global__ void k_to16r(const int32_t *__restrict__ S, int64_t lds, uint16_t *__restrict__ S16, int64_t ld16,
                        int64_t rows, int32_t cols) {
  const int64_t total = rows * (cols / 4);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / (cols / 4);
    const int32_t c4 = (int32_t)(i % (cols / 4)) * 4;
    const int4 v = *reinterpret_cast<const int4 *>(S + r * lds + c4);
    const uint32_t lo = (uint32_t)min(v.x, (int32_t)C16) | ((uint32_t)min(v.y, (int32_t)C16) << 16);
    const uint32_t hi = (uint32_t)min(v.z, (int32_t)C16) | ((uint32_t)min(v.w, (int32_t)C16) << 16);
    *reinterpret_cast<uint2 *>(S16 + r * ld16 + c4) = make_uint2(lo, hi);
  }
}

// the inverse (C16 -> INF)
__global__ void k_from16r(const uint16_t *__restrict__ S16, int64_t ld16, int32_t *__restrict__ S, int64_t lds,
                          int64_t rows, int32_t cols) {
  const int64_t total = rows * (cols / 4);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / (cols / 4);
    const int32_t c4 = (int32_t)(i % (cols / 4)) * 4;
    const uint2 v = *reinterpret_cast<const uint2 *>(S16 + r * ld16 + c4);
    auto f = [](uint32_t x) { return x == C16 ? INF : (int32_t)x; };
    *reinterpret_cast<int4 *>(S + r * lds + c4) = make_int4(f(v.x & 0xFFFFu), f(v.x >> 16), f(v.y & 0xFFFFu), f(v.y >> 16));
  }
}

// the assembled int32 pivot row block -> its capped u16 copy and (Pd non-null) the duplicated u32 copy;
// n = TILE * Np, n % 4 == 0
__global__ void k_prow_to16(const int32_t *__restrict__ P32, uint16_t *__restrict__ P16, uint32_t *__restrict__ Pd,
                            int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n / 4; i += (int64_t)gridDim.x * blockDim.x) {
    const int4 v = reinterpret_cast<const int4 *>(P32)[i];
    const uint32_t a = (uint32_t)min(v.x, (int32_t)C16), b = (uint32_t)min(v.y, (int32_t)C16);
    const uint32_t c = (uint32_t)min(v.z, (int32_t)C16), d = (uint32_t)min(v.w, (int32_t)C16);
    reinterpret_cast<uint2 *>(P16)[i] = make_uint2(a | (b << 16), c | (d << 16));
    if (Pd) reinterpret_cast<uint4 *>(Pd)[i] = make_uint4(a * 0x10001u, b * 0x10001u, c * 0x10001u, d * 0x10001u);
  }
}

// k_check16 over a rank's owned UPPER tiles (the authoritative ones; D is symmetric, so the ranks
// together cover every pair): a capped entry of a connected pair sets *flag = -1 (MIN-reducible)
__global__ void k_check16_list(const uint16_t *__restrict__ S16, int64_t ld16, const int32_t *__restrict__ orow,
                               int32_t nown, int32_t Np, const int32_t *__restrict__ lab, int32_t n_real,
                               int32_t *flag) {
  const int64_t per = (int64_t)TILE * (Np / 8);
  const int64_t total = (int64_t)nown * per;
  int found = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t lr = (int32_t)(i / per);
    const int64_t rem = i % per;
    const int32_t rr = (int32_t)(rem / (Np / 8)), c8 = (int32_t)(rem % (Np / 8)) * 8;
    const int32_t r = orow[lr] * TILE + rr;
    if (r >= n_real || c8 >= n_real || c8 < orow[lr] * TILE) continue;
    const uint4 v = *reinterpret_cast<const uint4 *>(S16 + ((int64_t)lr * TILE + rr) * ld16 + c8);
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint32_t x = (w[q >> 1] >> ((q & 1) * 16)) & 0xFFFFu;
      const int32_t c = c8 + q;
      if (x == C16 && c < n_real && (!lab || lab[r] == lab[c])) found = 1;
    }
  }
  if (__syncthreads_or(found) && threadIdx.x == 0) atomicMin(flag, -1);
}

// Closure of the 16-bit pivot tile (ld ldt) in place, packed like the tile kernel: thread (ty, tx)
// owns rows {ty*4 .. +3, 64 + ty*4 .. +3} as 4 row PAIRS and columns {tx*4 .. +3, 64 + tx*4 .. +3},
// c[p][q] = (T[i][j], T[i+1][j]); step kk reads row kk from shared memory -- it is also column kk, the
// tile being symmetric -- as the row-pair operand and, duplicated, as the column operand, so one
// VIADDMNMX.U16x2 relaxes two entries (values <= C16: sums <= 0xFFFE never wrap, results stay
// <= C16).  About 60 registers: it fits beside two CTAs of the tile kernel, which the lookahead
// needs (the int32-register closure took 108 x 256 registers, more than an SM has left then, so it
// waited for every rest-of-round launch to drain).
__global__ void __launch_bounds__(NT, 1) k_fw_phase1_16(uint16_t *T, int64_t ldt) {
  __shared__ __align__(16) uint16_t rowbuf[2][TILE];
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  uint32_t c[4][8];
#pragma unroll
  for (int p = 0; p < 4; ++p) {
    const int i = (p < 2 ? 0 : 64) + ty * 4 + (p & 1) * 2;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const uint2 v = *reinterpret_cast<const uint2 *>(T + (int64_t)i * ldt + h * 64 + tx * 4);
      const uint2 w = *reinterpret_cast<const uint2 *>(T + (int64_t)(i + 1) * ldt + h * 64 + tx * 4);
      c[p][h * 4 + 0] = __byte_perm(v.x, w.x, 0x5410);
      c[p][h * 4 + 1] = __byte_perm(v.x, w.x, 0x7632);
      c[p][h * 4 + 2] = __byte_perm(v.y, w.y, 0x5410);
      c[p][h * 4 + 3] = __byte_perm(v.y, w.y, 0x7632);
    }
  }
  if (threadIdx.x < TILE / 4)   // row 0
    reinterpret_cast<uint2 *>(rowbuf[0])[threadIdx.x] = reinterpret_cast<const uint2 *>(T)[threadIdx.x];
  __syncthreads();
  for (int kk = 0; kk < TILE; ++kk) {
    const uint16_t *rb = rowbuf[kk & 1];
    const uint2 alo = *reinterpret_cast<const uint2 *>(rb + ty * 4);        // rows ty*4 .. +3 (pairs)
    const uint2 ahi = *reinterpret_cast<const uint2 *>(rb + 64 + ty * 4);
    const uint2 blo = *reinterpret_cast<const uint2 *>(rb + tx * 4);        // columns tx*4 .. +3
    const uint2 bhi = *reinterpret_cast<const uint2 *>(rb + 64 + tx * 4);
    const uint32_t a[4] = {alo.x, alo.y, ahi.x, ahi.y};
    const uint32_t b[8] = {__byte_perm(blo.x, 0, 0x1010), __byte_perm(blo.x, 0, 0x3232),
                           __byte_perm(blo.y, 0, 0x1010), __byte_perm(blo.y, 0, 0x3232),
                           __byte_perm(bhi.x, 0, 0x1010), __byte_perm(bhi.x, 0, 0x3232),
                           __byte_perm(bhi.y, 0, 0x1010), __byte_perm(bhi.y, 0, 0x3232)};
#pragma unroll
    for (int p = 0; p < 4; ++p)
#pragma unroll
      for (int q = 0; q < 8; ++q) c[p][q] = __viaddmin_u16x2(a[p], b[q], c[p][q]);
    const int nk = kk + 1;   // its owner publishes row nk for the next step
    if (nk < TILE && ty == ((nk & 63) >> 2)) {
      const int p = ((nk & 3) >> 1) + (nk >= 64 ? 2 : 0), hi = nk & 1;
      uint16_t *wb = rowbuf[nk & 1];
#pragma unroll
      for (int pp = 0; pp < 4; ++pp) {
        if (pp == p) {
          const uint32_t sel = hi ? 0x7632 : 0x5410;
          *reinterpret_cast<uint2 *>(wb + tx * 4) =
              make_uint2(__byte_perm(c[pp][0], c[pp][1], sel), __byte_perm(c[pp][2], c[pp][3], sel));
          *reinterpret_cast<uint2 *>(wb + 64 + tx * 4) =
              make_uint2(__byte_perm(c[pp][4], c[pp][5], sel), __byte_perm(c[pp][6], c[pp][7], sel));
        }
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int p = 0; p < 4; ++p) {
    const int i = (p < 2 ? 0 : 64) + ty * 4 + (p & 1) * 2;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const uint32_t *cc = &c[p][h * 4];
      *reinterpret_cast<uint2 *>(T + (int64_t)i * ldt + h * 64 + tx * 4) =
          make_uint2(__byte_perm(cc[0], cc[1], 0x5410), __byte_perm(cc[2], cc[3], 0x5410));
      *reinterpret_cast<uint2 *>(T + (int64_t)(i + 1) * ldt + h * 64 + tx * 4) =
          make_uint2(__byte_perm(cc[0], cc[1], 0x7632), __byte_perm(cc[2], cc[3], 0x7632));
    }
  }
}

// Phases 2 and 3, packed: the same persistent TMA-ring structure as k_fw_tiles.  A^T chunks are 16-bit
// rows of the pivot row block (tmA: KC x 128 u16), B chunks rows of its duplicated copy Pd (tmB: KC x
// 128 u32).  Thread (ty, tx) owns rows {ty*4 .. +3, 64 + ty*4 .. +3} as 4 row PAIRS and columns
// {tx*4 .. +3, 64 + tx*4 .. +3}: c[r2][q] = (C[i][j], C[i+1][j]) packed, so one VIADDMNMX.U16x2
// c = min(c, a_pair + b_dup) does two min-plus.
struct TileJob16 {
  uint16_t *C;       // matrix holding the C tiles, leading dimension ldc (u16 elements)
  int64_t ldc;
  int32_t a_row0;    // row of the pivot row block inside tmA
  int32_t k, nt;
  int32_t mode;      // MODE_PIVOT_ROW, MODE_UPPER, MODE_CROSS, MODE_REST or MODE_LIST
  int32_t mirror;
  int64_t ntiles;
  // MODE_LIST (row-block sharded): as TileJob -- C holds the rank's owned tile rows only
  const int32_t *orow;
  const int64_t *opre;
  int32_t nown, mk, posk;
  unsigned long long *dbg;   // development (EAR_FW16_DBG): per-CTA %globaltimer at start / end, or null
  int32_t ti0;               // first tile row held by C (MODE_PIVOT_ROW on a standalone pivot row block: k)
  int32_t posk1;             // MODE_LIST_CROSS / _REST
  int32_t *counter;          // kDYN: {next tile, CTAs done}, zero at launch, reset by the last CTA
};

// LAR = 1: a ring stage is refilled by the LAST warp to finish consuming it (a shared counter) instead
// of thread 0 waiting on an 'empty' barrier at the start of each chunk (which ties warp 0 to the
// slowest warp every chunk).
template <int KC, int STAGES, int MINB, int UNR, int NTH = 256, int PFC = 0, int LAR = 0, int SPIN = 0,
          int DYN = 0, int HINT = 0>
struct Fw16Cfg {
  static constexpr int NCHUNK = TILE / KC;
  static constexpr int A_CHUNK = KC * TILE;   // u16 elements
  static constexpr int B_CHUNK = KC * TILE;   // u32 elements
  static constexpr int SMEM = STAGES * (A_CHUNK * 2 + B_CHUNK * 4) + 2 * STAGES * 8 + STAGES * 4 + 8;
  static constexpr int kKC = KC, kSTAGES = STAGES, kMINB = MINB, kUNR = UNR, kNTH = NTH, kPFC = PFC, kLAR = LAR;
  static constexpr int kSPIN = SPIN, kDYN = DYN, kHINT = HINT;
  static constexpr int RPH = 256 * 2 / NTH;   // row pairs per 64-row half owned by a thread (2 or 4)
};

__device__ __forceinline__ void decode16(const TileJob16 &J, int64_t idx, int &ti, int &tj, int &lr) {
  TileJob T{};
  T.k = J.k; T.nt = J.nt; T.mode = J.mode; T.ti0 = J.ti0;
  T.orow = J.orow; T.opre = J.opre; T.nown = J.nown; T.mk = J.mk; T.posk = J.posk; T.posk1 = J.posk1;
  decode_tile(T, idx, ti, tj, lr);
}

// Thread (ty, tx): columns {tx*4 .. +3, 64 + tx*4 .. +3}; rows {h*64 + ty*2*RPH + 2p, +1} for h = 0, 1 and
// p < RPH, i.e. 2*RPH row pairs (8 with 256 threads, 16 with 128).
template <class CF>
__global__ void __launch_bounds__(CF::kNTH, CF::kMINB)
    k_fw_tiles16(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, const TileJob16 J) {
  constexpr int KC = CF::kKC, NCHUNK = CF::NCHUNK, STAGES = CF::kSTAGES, NTH = CF::kNTH, RPH = CF::RPH;
  constexpr int NRP = 2 * RPH;   // row pairs per thread
  extern __shared__ __align__(128) uint8_t smem16[];
  uint16_t *sA = reinterpret_cast<uint16_t *>(smem16);                        // [STAGES][KC][TILE] u16
  uint32_t *sB = reinterpret_cast<uint32_t *>(sA + STAGES * CF::A_CHUNK);     // [STAGES][KC][TILE] u32
  uint64_t *full = reinterpret_cast<uint64_t *>(sB + STAGES * CF::B_CHUNK);
  uint64_t *empty = full + STAGES;
  int32_t *cnt = reinterpret_cast<int32_t *>(empty + STAGES);   // LAR: warps done with the stage
  const int tid = threadIdx.x, lane = tid & 31;
  const int tx = tid & 15, ty = tid >> 4;
  if (J.dbg && tid == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    J.dbg[3 * blockIdx.x] = t;
    J.dbg[3 * blockIdx.x + 2] = smid;
  }

  const int my_tiles = J.ntiles > (int64_t)blockIdx.x ? (int)((J.ntiles - 1 - blockIdx.x) / gridDim.x + 1) : 0;
  const int total_chunks = my_tiles * NCHUNK;
  int issued = 0;
  auto tile_of = [&](int it, int &ti, int &tj, int &lr) { decode16(J, blockIdx.x + (int64_t)it * gridDim.x, ti, tj, lr); };
  auto issue = [&](int c, int st) {   // chunk c into stage st
    int pti, ptj, plr;
    tile_of(c / NCHUNK, pti, ptj, plr);
    const int kc = c % NCHUNK;
    mbar_arrive_tx(&full[st], CF::A_CHUNK * 2 + CF::B_CHUNK * 4);
    tma_load_2d(sA + st * CF::A_CHUNK, &tmA, pti * TILE, J.a_row0 + kc * KC, &full[st]);
    tma_load_2d(sB + st * CF::B_CHUNK, &tmB, ptj * TILE, kc * KC, &full[st]);
  };
  auto produce = [&](int upto) {
    while (issued < upto) {
      const int st = issued % STAGES;
      if (issued >= STAGES) mbar_wait(&empty[st], (uint32_t)((issued / STAGES - 1) & 1));
      int pti, ptj, plr;
      tile_of(issued / NCHUNK, pti, ptj, plr);
      const int kc = issued % NCHUNK;
      mbar_arrive_tx(&full[st], CF::A_CHUNK * 2 + CF::B_CHUNK * 4);
      tma_load_2d(sA + st * CF::A_CHUNK, &tmA, pti * TILE, J.a_row0 + kc * KC, &full[st]);
      tma_load_2d(sB + st * CF::B_CHUNK, &tmB, ptj * TILE, kc * KC, &full[st]);
      ++issued;
    }
  };
  if (tid == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], NTH / 32);
      cnt[s] = 0;
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&tmA)) : "memory");
    asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&tmB)) : "memory");
  }
  __syncthreads();
  if (tid == 0 && my_tiles > 0) {
    if (CF::kLAR) {
      for (int c = 0; c < STAGES && c < total_chunks; ++c) issue(c, c);
    } else {
      produce(total_chunks < STAGES ? total_chunks : STAGES);
    }
  }

  auto row_of = [&](int r2) { return (r2 < RPH ? 0 : 64) + ty * 2 * RPH + (r2 % RPH) * 2; };
  int g = 0;
  for (int it = 0; it < my_tiles; ++it) {
    int ti, tj, lr;
    tile_of(it, ti, tj, lr);
    uint32_t c[NRP][8];
    uint16_t *Ct = J.C + (int64_t)lr * TILE * J.ldc + (int64_t)tj * TILE;
#pragma unroll
    for (int r2 = 0; r2 < NRP; ++r2) {
      const int i = row_of(r2);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const uint2 v = *reinterpret_cast<const uint2 *>(Ct + (int64_t)i * J.ldc + h * 64 + tx * 4);
        const uint2 w = *reinterpret_cast<const uint2 *>(Ct + (int64_t)(i + 1) * J.ldc + h * 64 + tx * 4);
        c[r2][h * 4 + 0] = __byte_perm(v.x, w.x, 0x5410);
        c[r2][h * 4 + 1] = __byte_perm(v.x, w.x, 0x7632);
        c[r2][h * 4 + 2] = __byte_perm(v.y, w.y, 0x5410);
        c[r2][h * 4 + 3] = __byte_perm(v.y, w.y, 0x7632);
      }
    }
    if (CF::kPFC && it + 1 < my_tiles) {   // pull the next tile's C rows into L2 while this one computes
      int nti, ntj, nlr;
      tile_of(it + 1, nti, ntj, nlr);
      const uint16_t *Cn = J.C + (int64_t)nlr * TILE * J.ldc + (int64_t)ntj * TILE;
      // 128 rows x 256 B: one 128-byte line per (row, half), spread over the CTA's threads
      for (int l = tid; l < 2 * TILE; l += NTH)
        asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(Cn + (int64_t)(l >> 1) * J.ldc + (l & 1) * 64));
    }
#pragma unroll 1
    for (int kc = 0; kc < NCHUNK; ++kc, ++g) {
      if (!CF::kLAR && tid == 0) produce(g + STAGES < total_chunks ? g + STAGES : total_chunks);
      const int st = g % STAGES;
      if (CF::kSPIN) mbar_wait_spin(&full[st], (uint32_t)((g / STAGES) & 1));
      else mbar_wait(&full[st], (uint32_t)((g / STAGES) & 1));
      const uint16_t *a_s = sA + st * CF::A_CHUNK;
      const uint32_t *b_s = sB + st * CF::B_CHUNK;
#pragma unroll CF::kUNR
      for (int kk = 0; kk < KC; ++kk) {
        uint32_t a[NRP];
        if (RPH == 2) {
          const uint2 alo = *reinterpret_cast<const uint2 *>(a_s + kk * TILE + ty * 4);
          const uint2 ahi = *reinterpret_cast<const uint2 *>(a_s + kk * TILE + 64 + ty * 4);
          a[0] = alo.x; a[1] = alo.y; a[RPH] = ahi.x; a[RPH + 1] = ahi.y;
        } else {
          const uint4 alo = *reinterpret_cast<const uint4 *>(a_s + kk * TILE + ty * 8);
          const uint4 ahi = *reinterpret_cast<const uint4 *>(a_s + kk * TILE + 64 + ty * 8);
          a[0] = alo.x; a[1] = alo.y; a[2] = alo.z; a[3] = alo.w;
          a[RPH] = ahi.x; a[RPH + 1] = ahi.y; a[RPH + 2] = ahi.z; a[RPH + 3] = ahi.w;
        }
        const uint4 blo = *reinterpret_cast<const uint4 *>(b_s + kk * TILE + tx * 4);
        const uint4 bhi = *reinterpret_cast<const uint4 *>(b_s + kk * TILE + 64 + tx * 4);
        const uint32_t b[8] = {blo.x, blo.y, blo.z, blo.w, bhi.x, bhi.y, bhi.z, bhi.w};
#pragma unroll
        for (int r2 = 0; r2 < NRP; ++r2)
#pragma unroll
          for (int q = 0; q < 8; ++q) c[r2][q] = __viaddmin_u16x2(a[r2], b[q], c[r2][q]);
      }
      __syncwarp();
      if (CF::kLAR) {
        if (lane == 0) {
          __threadfence_block();
          if (atomicAdd(&cnt[st], 1) == NTH / 32 - 1) {   // the last reader of this stage refills it
            cnt[st] = 0;
            __threadfence_block();
            asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
            if (g + STAGES < total_chunks) issue(g + STAGES, st);
          }
        }
      } else if (lane == 0) {
        mbar_arrive(&empty[st]);
      }
    }
#pragma unroll
    for (int r2 = 0; r2 < NRP; ++r2) {
      const int i = row_of(r2);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const uint32_t *cc = &c[r2][h * 4];
        *reinterpret_cast<uint2 *>(Ct + (int64_t)i * J.ldc + h * 64 + tx * 4) =
            make_uint2(__byte_perm(cc[0], cc[1], 0x5410), __byte_perm(cc[2], cc[3], 0x5410));
        *reinterpret_cast<uint2 *>(Ct + (int64_t)(i + 1) * J.ldc + h * 64 + tx * 4) =
            make_uint2(__byte_perm(cc[0], cc[1], 0x7632), __byte_perm(cc[2], cc[3], 0x7632));
      }
    }
    if (J.mirror && ti != tj) {
      uint16_t *Mt = J.C + (int64_t)tj * TILE * J.ldc + (int64_t)ti * TILE;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const int j = (q < 4 ? 0 : 64) + tx * 4 + (q & 3);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          if (RPH == 2) {
            *reinterpret_cast<uint2 *>(Mt + (int64_t)j * J.ldc + h * 64 + ty * 4) = make_uint2(c[h * 2][q], c[h * 2 + 1][q]);
          } else {
            *reinterpret_cast<uint4 *>(Mt + (int64_t)j * J.ldc + h * 64 + ty * 8) =
                make_uint4(c[h * 4][q], c[h * 4 + 1][q], c[h * 4 + 2][q], c[h * 4 + 3][q]);
          }
        }
      }
    }
  }
  if (J.dbg) {
    __syncthreads();
    if (tid == 0) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      J.dbg[3 * blockIdx.x + 1] = t;
    }
  }
}

// Dynamically scheduled version of k_fw_tiles16 (CF::kDYN): a CTA takes its next tile from a global
// counter when it issues that tile's first TMA chunk, instead of the static blockIdx + it * grid
// assignment.  Measured with the static assignment (tools/fw16_cta_times.py): all CTAs start
// together but end between 43 % and 100 % of the launch -- the SM's warp scheduler favours its oldest
// CTA, so the three CTAs of an SM run at different speeds and each SM spends the last part of every
// launch with one or two of them (2.15 resident CTAs on average).  With the counter, fast CTAs simply
// take more tiles.  The tile of a CTA's tile sequence number q is published in tslot[q & 1] (tagged
// with q) by the thread that issues its first chunk; the ring depth (2) never exceeds the chunks per
// tile (4), so a slot is rewritten only after every warp has read it.  The last CTA to finish resets
// the counter pair for the next launch on the same stream.
template <class CF>
__global__ void __launch_bounds__(CF::kNTH, CF::kMINB)
    k_fw_tiles16_dyn(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                     const TileJob16 J) {
  constexpr int KC = CF::kKC, NCHUNK = CF::NCHUNK, STAGES = CF::kSTAGES, NTH = CF::kNTH, RPH = CF::RPH;
  constexpr int NRP = 2 * RPH, NW = NTH / 32;
  static_assert(NCHUNK >= STAGES, "tile slots are rewritten only after every warp has read them");
  constexpr int32_t NONE = 0xFFFFF;
  extern __shared__ __align__(128) uint8_t smem16[];
  uint16_t *sA = reinterpret_cast<uint16_t *>(smem16);
  uint32_t *sB = reinterpret_cast<uint32_t *>(sA + STAGES * CF::A_CHUNK);
  uint64_t *full = reinterpret_cast<uint64_t *>(sB + STAGES * CF::B_CHUNK);
  int32_t *cnt = reinterpret_cast<int32_t *>(full + 2 * STAGES);   // [STAGES] warps done with the stage
  int32_t *tslot = cnt + STAGES;                                   // [2] (q << 20) | tile
  const int tid = threadIdx.x, lane = tid & 31;
  const int tx = tid & 15, ty = tid >> 4;
  if (J.dbg && tid == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    J.dbg[3 * blockIdx.x] = t;
    J.dbg[3 * blockIdx.x + 2] = smid;
  }
  // chunk c of this CTA's sequence into stage st (one thread)
  auto issue = [&](int c, int st) {
    const int q = c / NCHUNK, kc = c % NCHUNK;
    int32_t t;
    if (kc == 0) {
      const int32_t tt = atomicAdd(J.counter, 1);
      t = tt < J.ntiles ? tt : -1;
      tslot[q & 1] = (q << 20) | (t < 0 ? NONE : t);
      __threadfence_block();
    } else {
      const int32_t v = tslot[q & 1] & NONE;
      t = v == NONE ? -1 : v;
    }
    if (t < 0) {   // no tile: complete the phase without data so that the waiters see the end
      mbar_arrive(&full[st]);
      return;
    }
    int pti, ptj, plr;
    decode16(J, t, pti, ptj, plr);
    mbar_arrive_tx(&full[st], CF::A_CHUNK * 2 + CF::B_CHUNK * 4);
    if (CF::kHINT) {   // the pivot row block stays in L2 while the C tiles stream through it
      uint64_t pol;
      asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
      tma_load_2d_hint(sA + st * CF::A_CHUNK, &tmA, pti * TILE, J.a_row0 + kc * KC, &full[st], pol);
      tma_load_2d_hint(sB + st * CF::B_CHUNK, &tmB, ptj * TILE, kc * KC, &full[st], pol);
    } else {
      tma_load_2d(sA + st * CF::A_CHUNK, &tmA, pti * TILE, J.a_row0 + kc * KC, &full[st]);
      tma_load_2d(sB + st * CF::B_CHUNK, &tmB, ptj * TILE, kc * KC, &full[st]);
    }
  };
  if (tid == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      cnt[s] = 0;
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&tmA)) : "memory");
    asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&tmB)) : "memory");
  }
  __syncthreads();
  if (tid == 0)
    for (int c = 0; c < STAGES; ++c) issue(c, c);

  auto row_of = [&](int r2) { return (r2 < RPH ? 0 : 64) + ty * 2 * RPH + (r2 % RPH) * 2; };
  int g = 0;
  for (int q = 0;; ++q) {
    mbar_wait(&full[g % STAGES], (uint32_t)((g / STAGES) & 1));
    const int32_t v = tslot[q & 1] & NONE;
    if (v == NONE) break;
    int ti, tj, lr;
    decode16(J, v, ti, tj, lr);
    uint32_t c[NRP][8];
    uint16_t *Ct = J.C + (int64_t)lr * TILE * J.ldc + (int64_t)tj * TILE;
#pragma unroll
    for (int r2 = 0; r2 < NRP; ++r2) {
      const int i = row_of(r2);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const uint2 *pa = reinterpret_cast<const uint2 *>(Ct + (int64_t)i * J.ldc + h * 64 + tx * 4);
        const uint2 *pb = reinterpret_cast<const uint2 *>(Ct + (int64_t)(i + 1) * J.ldc + h * 64 + tx * 4);
        const uint2 a = CF::kHINT ? __ldcs(pa) : *pa;
        const uint2 b = CF::kHINT ? __ldcs(pb) : *pb;
        c[r2][h * 4 + 0] = __byte_perm(a.x, b.x, 0x5410);
        c[r2][h * 4 + 1] = __byte_perm(a.x, b.x, 0x7632);
        c[r2][h * 4 + 2] = __byte_perm(a.y, b.y, 0x5410);
        c[r2][h * 4 + 3] = __byte_perm(a.y, b.y, 0x7632);
      }
    }
#pragma unroll 1
    for (int kc = 0; kc < NCHUNK; ++kc, ++g) {
      const int st = g % STAGES;
      if (kc > 0) mbar_wait(&full[st], (uint32_t)((g / STAGES) & 1));
      if (CF::kPFC && kc == NCHUNK - 1) {   // the next tile, once published: its C rows into L2
        const int32_t nv = tslot[(q + 1) & 1];
        if ((nv >> 20) == q + 1 && (nv & NONE) != NONE) {
          int nti, ntj, nlr;
          decode16(J, nv & NONE, nti, ntj, nlr);
          const uint16_t *Cn = J.C + (int64_t)nlr * TILE * J.ldc + (int64_t)ntj * TILE;
          for (int l = tid; l < 2 * TILE; l += NTH)
            asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(Cn + (int64_t)(l >> 1) * J.ldc + (l & 1) * 64));
        }
      }
      const uint16_t *a_s = sA + st * CF::A_CHUNK;
      const uint32_t *b_s = sB + st * CF::B_CHUNK;
#pragma unroll CF::kUNR
      for (int kk = 0; kk < KC; ++kk) {
        uint32_t a[NRP];
        if (RPH == 2) {
          const uint2 alo = *reinterpret_cast<const uint2 *>(a_s + kk * TILE + ty * 4);
          const uint2 ahi = *reinterpret_cast<const uint2 *>(a_s + kk * TILE + 64 + ty * 4);
          a[0] = alo.x; a[1] = alo.y; a[RPH] = ahi.x; a[RPH + 1] = ahi.y;
        } else {
          const uint4 alo = *reinterpret_cast<const uint4 *>(a_s + kk * TILE + ty * 8);
          const uint4 ahi = *reinterpret_cast<const uint4 *>(a_s + kk * TILE + 64 + ty * 8);
          a[0] = alo.x; a[1] = alo.y; a[2] = alo.z; a[3] = alo.w;
          a[RPH] = ahi.x; a[RPH + 1] = ahi.y; a[RPH + 2] = ahi.z; a[RPH + 3] = ahi.w;
        }
        const uint4 blo = *reinterpret_cast<const uint4 *>(b_s + kk * TILE + tx * 4);
        const uint4 bhi = *reinterpret_cast<const uint4 *>(b_s + kk * TILE + 64 + tx * 4);
        const uint32_t b[8] = {blo.x, blo.y, blo.z, blo.w, bhi.x, bhi.y, bhi.z, bhi.w};
#pragma unroll
        for (int r2 = 0; r2 < NRP; ++r2)
#pragma unroll
          for (int qq = 0; qq < 8; ++qq) c[r2][qq] = __viaddmin_u16x2(a[r2], b[qq], c[r2][qq]);
      }
      __syncwarp();
      if (lane == 0) {
        __threadfence_block();
        if (atomicAdd(&cnt[st], 1) == NW - 1) {   // the last reader of this stage refills it
          cnt[st] = 0;
          __threadfence_block();
          asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
          issue(g + STAGES, st);
        }
      }
    }
#pragma unroll
    for (int r2 = 0; r2 < NRP; ++r2) {
      const int i = row_of(r2);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const uint32_t *cc = &c[r2][h * 4];
        uint2 *qa = reinterpret_cast<uint2 *>(Ct + (int64_t)i * J.ldc + h * 64 + tx * 4);
        uint2 *qb = reinterpret_cast<uint2 *>(Ct + (int64_t)(i + 1) * J.ldc + h * 64 + tx * 4);
        const uint2 va = make_uint2(__byte_perm(cc[0], cc[1], 0x5410), __byte_perm(cc[2], cc[3], 0x5410));
        const uint2 vb = make_uint2(__byte_perm(cc[0], cc[1], 0x7632), __byte_perm(cc[2], cc[3], 0x7632));
        if (CF::kHINT) { __stcs(qa, va); __stcs(qb, vb); } else { *qa = va; *qb = vb; }
      }
    }
    if (J.mirror && ti != tj) {
      uint16_t *Mt = J.C + (int64_t)tj * TILE * J.ldc + (int64_t)ti * TILE;
#pragma unroll
      for (int qq = 0; qq < 8; ++qq) {
        const int j = (qq < 4 ? 0 : 64) + tx * 4 + (qq & 3);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          if (RPH == 2) {
            *reinterpret_cast<uint2 *>(Mt + (int64_t)j * J.ldc + h * 64 + ty * 4) = make_uint2(c[h * 2][qq], c[h * 2 + 1][qq]);
          } else {
            *reinterpret_cast<uint4 *>(Mt + (int64_t)j * J.ldc + h * 64 + ty * 8) =
                make_uint4(c[h * 4][qq], c[h * 4 + 1][qq], c[h * 4 + 2][qq], c[h * 4 + 3][qq]);
          }
        }
      }
    }
  }
  __syncthreads();
  if (tid == 0) {
    if (J.dbg) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      J.dbg[3 * blockIdx.x + 1] = t;
    }
    __threadfence();
    if (atomicAdd(J.counter + 1, 1) == (int)gridDim.x - 1) {   // the last CTA resets the pair
      J.counter[0] = 0;
      J.counter[1] = 0;
      __threadfence();
    }
  }
}

// connected-component labels (min vertex id) of the reduced graph by hooking + pointer jumping
__global__ void k_cc_init(int32_t *lab, int32_t n) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    lab[v] = (int32_t)v;
}
__global__ void k_cc_hook16(const int32_t *u, const int32_t *v, int64_t E, int32_t *lab, int32_t *changed) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < E; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t a = lab[u[i]], b = lab[v[i]];
    if (a != b) {
      const int32_t hi = max(a, b), lo = min(a, b);
      if (atomicMin(&lab[hi], lo) > lo) *changed = 1;
    }
  }
}
__global__ void k_cc_jump16(int32_t *lab, int32_t n) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    int32_t l = lab[v];
    while (lab[l] != l) l = lab[l];
    lab[v] = l;
  }
}

int g_num_sms = 0;
PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;

// 2-D tensor map over rows x cols (leading dimension ld elements of elem bytes) with a box_rows x 128 box
ear_status_t make_map_t(CUtensorMap *map, CUtensorMapDataType dt, int elem, const void *base, int64_t rows,
                        int64_t cols, int64_t ld, int box_rows) {
  if (!g_encode) {
    cudaDriverEntryPointQueryResult q;
    void *fn = nullptr;
    EAR_CUDA_TRY(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    if (!fn || q != cudaDriverEntryPointSuccess) {
      set_error("cuTensorMapEncodeTiled unavailable");
      return EAR_ECUDA;
    }
    g_encode = (PFN_cuTensorMapEncodeTiled_v12000)fn;
  }
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)ld * elem};
  cuuint32_t box[2] = {(cuuint32_t)TILE, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = g_encode(map, dt, 2, const_cast<void *>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d) rows=%lld cols=%lld ld=%lld", (int)r, (long long)rows,
              (long long)cols, (long long)ld);
    return EAR_ECUDA;
  }
  return EAR_OK;
}

ear_status_t make_map(CUtensorMap *map, const int32_t *base, int64_t rows, int64_t cols, int64_t ld, int box_rows) {
  return make_map_t(map, CU_TENSOR_MAP_DATA_TYPE_INT32, 4, base, rows, cols, ld, box_rows);
}

// The tile kernel's configuration, chosen by measurement on the B200 (cfg4, phase-3 share of the
// VIADDMNMX peak; profiles/r01_fw_variants.txt): 64-deep k-chunks, a 2-stage TMA ring (128 KB), C
// straight into registers, one 256-thread CTA per SM (161 registers, no spills), kk unrolled 16x.
using FwTile = FwCfg<64, 2, 1, 16>;

int fw_kc() { return FwTile::KC; }

template <class CF>
ear_status_t launch_cfg(const CUtensorMap &map, const TileJob &J, int64_t nblocks, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    EAR_CUDA_TRY(cudaFuncSetAttribute(k_fw_tiles<CF>, cudaFuncAttributeMaxDynamicSharedMemorySize, CF::SMEM));
    attr = true;
  }
  int per_sm = 0;
  EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_fw_tiles<CF>, NT, CF::SMEM));
  if (per_sm < 1) per_sm = 1;
  const int64_t grid = std::min<int64_t>(nblocks, (int64_t)g_num_sms * per_sm);   // persistent
  EAR_LAUNCH(k_fw_tiles<CF>, (unsigned)grid, NT, CF::SMEM, st)(map, J);
  return EAR_OK;
}

ear_status_t launch_tiles(const CUtensorMap &map, TileJob J, int64_t nblocks, cudaStream_t st) {
  if (!g_num_sms) {
    int dev = 0;
    EAR_CUDA_TRY(cudaGetDevice(&dev));
    EAR_CUDA_TRY(cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev));
  }
  if (nblocks <= 0) return EAR_OK;
  J.ntiles = nblocks;
  return launch_cfg<FwTile>(map, J, nblocks, st);
}


// Packed 16-bit tile kernel configuration, chosen by tools/sweep_fw16.py on the B200 (cfg4, 17
// variants, profiles/r01_fw16_variants.jsonl): 128 threads with 16 x 8 values each, 32-deep k-chunks,
// a 2-stage TMA ring (48 KB), 3 CTAs per SM, kk unrolled 16x; then (tools/lab_fw16_variant.sh,
// profiles/r01u_fw16_refill.jsonl) last-arriver refills of the ring and an L2 prefetch of the next
// C tile: 475.3 -> 471.6 ms on cfg4's plain FW (3-stage rings and 16-deep chunks measured slower);
// then dynamic tile scheduling (k_fw_tiles16_dyn, the CTAs of an SM run at different speeds) and 4 CTA
// slots left to the lookahead's pivot chain: 472.7 -> 445.9 ms (profiles/r01y_fw16_dyn.jsonl).
using Fw16Tile = Fw16Cfg<32, 2, 3, 16, 128, 0, 1, 0, 1>;   // dynamic tile scheduling (k_fw_tiles16_dyn)
using Fw16TileL = Fw16Cfg<32, 2, 3, 16, 128, 0, 1>;
using Fw16TileL4 = Fw16Cfg<16, 4, 3, 16, 128, 0, 1>;
using Fw16TileL3 = Fw16Cfg<32, 3, 3, 16, 128, 0, 1>;
using Fw16TileLP = Fw16Cfg<32, 2, 3, 16, 128, 1, 1>;   // the static default before the tile counter
using Fw16TileL3P = Fw16Cfg<32, 3, 3, 16, 128, 1, 1>;
using Fw16TileS = Fw16Cfg<32, 2, 3, 16, 128, 1, 1, 1>;
using Fw16TileS3 = Fw16Cfg<32, 3, 3, 16, 128, 1, 1, 1>;
using Fw16TileD = Fw16Cfg<32, 2, 3, 16, 128, 1, 1, 0, 1>;
using Fw16TileD0 = Fw16Cfg<32, 2, 3, 16, 128, 0, 1, 0, 1>;
using Fw16TileD3 = Fw16Cfg<32, 3, 3, 16, 128, 0, 1, 0, 1>;
using Fw16TileD16 = Fw16Cfg<16, 4, 3, 16, 128, 0, 1, 0, 1>;
using Fw16TileD2x4 = Fw16Cfg<32, 4, 2, 16, 128, 0, 1, 0, 1>;
using Fw16TileD2x3 = Fw16Cfg<32, 3, 2, 16, 128, 0, 1, 0, 1>;
using Fw16TileDH = Fw16Cfg<32, 2, 3, 16, 128, 0, 1, 0, 1, 1>;

// development knobs (tools/): EAR_FW16_LOOKAHEAD=0 disables the lookahead, EAR_FW16_RESERVE sets the
// CTA slots the rest-of-round launch leaves free for the next round's pivot work (default 4: with the
// persistent dynamically scheduled kernel no slot frees up before the launch drains; measured best,
// profiles/r01y_fw16_dyn.jsonl), EAR_FW16_PRIO=0 gives the side stream normal priority
int env_int(const char *name, int dflt) {
  const char *e = getenv(name);
  return e ? atoi(e) : dflt;
}

// the dynamic kernel's counter pair for launches on stream st: one pair per (device, stream), zeroed
// once and reset by each launch's last CTA, so launches on one stream reuse it in order
int32_t *dyn_counter(cudaStream_t st) {
  static std::vector<std::pair<std::pair<int, cudaStream_t>, int32_t *>> pairs;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return nullptr;
  for (auto &p : pairs)
    if (p.first.first == dev && p.first.second == st) return p.second;
  int32_t *c = nullptr;
  if (cudaMalloc((void **)&c, 2 * sizeof(int32_t)) != cudaSuccess || cudaMemset(c, 0, 2 * sizeof(int32_t)) != cudaSuccess)
    return nullptr;
  pairs.push_back({{dev, st}, c});
  return c;
}

template <class CF>
ear_status_t launch16_cfg(const CUtensorMap &mA, const CUtensorMap &mB, TileJob16 J, int64_t nblocks, cudaStream_t st,
                          int reserve) {
  auto kern = CF::kDYN ? k_fw_tiles16_dyn<CF> : k_fw_tiles16<CF>;
  static bool attr = false;
  if (!attr) {
    EAR_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, CF::SMEM));
    attr = true;
  }
  if (CF::kDYN) {
    J.counter = dyn_counter(st);
    if (!J.counter) {
      set_error("fw16: no tile counter");
      return EAR_ECUDA;
    }
  }
  int per_sm = 0;
  EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, CF::kNTH, CF::SMEM));
  if (per_sm < 1) per_sm = 1;
  J.ntiles = nblocks;
  const int64_t grid = std::min<int64_t>(nblocks, std::max<int64_t>(1, (int64_t)g_num_sms * per_sm - reserve));
  // EAR_FW16_DBG=N (development): per-CTA start / end times and SM of the N-th launch, to stderr
  static const int dbg_at = env_int("EAR_FW16_DBG", -1);
  static int nlaunch = 0;
  const bool dbg = dbg_at >= 0 && nlaunch++ == dbg_at;
  if (dbg) EAR_CUDA_TRY(cudaMalloc((void **)&J.dbg, sizeof(unsigned long long) * 3 * grid));
  EAR_LAUNCH(kern, (unsigned)grid, CF::kNTH, CF::SMEM, st)(mA, mB, J);
  if (dbg) {
    std::vector<unsigned long long> h(3 * grid);
    EAR_CUDA_TRY(cudaStreamSynchronize(st));
    EAR_CUDA_TRY(cudaMemcpy(h.data(), J.dbg, sizeof(unsigned long long) * 3 * grid, cudaMemcpyDeviceToHost));
    cudaFree(J.dbg);
    unsigned long long t0 = ~0ull;
    for (int64_t b = 0; b < grid; ++b) t0 = std::min(t0, h[3 * b]);
    fprintf(stderr, "FW16DBG launch %d grid %lld tiles %lld per_sm %d\n", dbg_at, (long long)grid, (long long)nblocks, per_sm);
    for (int64_t b = 0; b < grid; ++b)
      fprintf(stderr, "FW16DBG %lld %llu %llu %llu\n", (long long)b, h[3 * b] - t0, h[3 * b + 1] - t0, h[3 * b + 2]);
  }
  return EAR_OK;
}

int fw16_kc() {
  const int v = env_int("EAR_FW16_VARIANT", 0);
  return v == 2 ? Fw16TileL4::kKC : v == 11 ? Fw16TileD16::kKC : Fw16Tile::kKC;
}

// EAR_FW16_VARIANT (development knob, tools/lab_fw16_*.sh): 0 = Fw16Tile; static tile assignment:
// 1 = last-arriver refill, 2 = 4-stage ring of 16-deep chunks, 3 = 3-stage ring, 4 = refill + C prefetch
// (the static default before), 5 = 3-stage + prefetch, 6/7 = polling waits; 8 = dynamic + C prefetch
template <class CF>
ear_status_t launch16(const CUtensorMap &mA, const CUtensorMap &mB, TileJob16 J, int64_t nblocks, cudaStream_t st,
                      int reserve = 0) {
  if (nblocks <= 0) return EAR_OK;
  static const int variant = env_int("EAR_FW16_VARIANT", 0);
  if (variant == 1) return launch16_cfg<Fw16TileL>(mA, mB, J, nblocks, st, reserve);
  if (variant == 2) return launch16_cfg<Fw16TileL4>(mA, mB, J, nblocks, st, reserve);
  if (variant == 3) return launch16_cfg<Fw16TileL3>(mA, mB, J, nblocks, st, reserve);
  if (variant == 4) return launch16_cfg<Fw16TileLP>(mA, mB, J, nblocks, st, reserve);
  if (variant == 5) return launch16_cfg<Fw16TileL3P>(mA, mB, J, nblocks, st, reserve);
  if (variant == 6) return launch16_cfg<Fw16TileS>(mA, mB, J, nblocks, st, reserve);
  if (variant == 7) return launch16_cfg<Fw16TileS3>(mA, mB, J, nblocks, st, reserve);
  if (variant == 8) return launch16_cfg<Fw16TileD>(mA, mB, J, nblocks, st, reserve);
  if (variant == 9) return launch16_cfg<Fw16TileD0>(mA, mB, J, nblocks, st, reserve);
  if (variant == 10) return launch16_cfg<Fw16TileD3>(mA, mB, J, nblocks, st, reserve);
  if (variant == 11) return launch16_cfg<Fw16TileD16>(mA, mB, J, nblocks, st, reserve);
  if (variant == 12) return launch16_cfg<Fw16TileD2x4>(mA, mB, J, nblocks, st, reserve);
  if (variant == 13) return launch16_cfg<Fw16TileD2x3>(mA, mB, J, nblocks, st, reserve);
  if (variant == 14) return launch16_cfg<Fw16TileDH>(mA, mB, J, nblocks, st, reserve);
  return launch16_cfg<CF>(mA, mB, J, nblocks, st, reserve);
}

int grid_for(int64_t n) { return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 16)); }

// CTA slots the rest-of-round launch leaves to the next round's pivot chain.  The persistent,
// dynamically scheduled tile kernel frees no slot before it drains, so the chain's phase-2 tiles (one
// pivot row, p2 tiles) run on the reserved slots alongside the rest (rest tiles): enough slots that
// they finish no later, p2 / R <= rest / (slots - R).  EAR_FW16_RESERVE overrides (measured on cfg4's
// single-GPU FW: 4 best, profiles/r01y_fw16_dyn.jsonl -- the rule gives 4 there, 5 on the re-reduced
// BCC root piece and ~27 for a rank of 8, whose rest is 8x smaller; profiles/r01z_rank_timing_cfg4.jsonl).
int lookahead_reserve(int64_t rest, int64_t p2) {
  const int forced = env_int("EAR_FW16_RESERVE", -1);
  if (forced >= 0) return forced;
  const int64_t slots = (int64_t)std::max(g_num_sms, 1) * 3;
  const int64_t r = (slots * p2 + rest + p2 - 1) / std::max<int64_t>(rest + p2, 1);
  return (int)std::min<int64_t>(std::max<int64_t>(r, 1), slots / 2);
}

// the lookahead's side stream and events of the current device (created once, shared by the single-GPU
// and the sharded packed FW; one FW call at a time per device)
ear_status_t side_stream(cudaStream_t *side, cudaEvent_t *ev_cross, cudaEvent_t *ev_pivot) {
  static cudaStream_t sides[64] = {};
  static cudaEvent_t crosses[64] = {}, pivots[64] = {};
  int dev = 0;
  EAR_CUDA_TRY(cudaGetDevice(&dev));
  if (dev < 0 || dev >= 64) { set_error("side_stream: device %d out of range", dev); return EAR_EINVAL; }
  if (!sides[dev]) {
    int lo = 0, hi = 0;   // the pivot work gets the highest priority: its CTAs take the first free slots
    EAR_CUDA_TRY(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    EAR_CUDA_TRY(cudaStreamCreateWithPriority(&sides[dev], cudaStreamNonBlocking, env_int("EAR_FW16_PRIO", 1) ? hi : lo));
    EAR_CUDA_TRY(cudaEventCreateWithFlags(&crosses[dev], cudaEventDisableTiming));
    EAR_CUDA_TRY(cudaEventCreateWithFlags(&pivots[dev], cudaEventDisableTiming));
  }
  *side = sides[dev];
  *ev_cross = crosses[dev];
  *ev_pivot = pivots[dev];
  return EAR_OK;
}

// Cap precheck of the packed FW: one single-source SSSP row of reduced vertex 0 on a helper stream,
// its eccentricity (a lower bound on the largest finite distance) read back asynchronously.  start()
// does nothing without a plan, for a small FW (< 64 tiles) or with EAR_FW16_PRECHECK=0; hopeless()
// waits for the row and says whether it reached the cap.  The row is exact and deterministic, so every
// rank of a sharded FW takes the same decision without a collective.
struct Precheck {
  cudaStream_t hs = nullptr;
  cudaEvent_t ev = nullptr;
  int32_t *row = nullptr;
  bool on = false;
  static int32_t *host() {   // pinned, one per process (one FW at a time)
    static int32_t *h = nullptr;
    if (!h && cudaHostAlloc((void **)&h, sizeof(int32_t), cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
      h = nullptr;
    return h;
  }
  void start(ear_plan_s *plan, int32_t Np, int32_t n_real, int nt) {
    if (!plan || nt < 64 || env_int("EAR_FW16_PRECHECK", 1) == 0 || !host()) return;
    on = cudaStreamCreateWithFlags(&hs, cudaStreamNonBlocking) == cudaSuccess &&
         cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) == cudaSuccess &&
         cudaMallocAsync((void **)&row, sizeof(int32_t) * ((size_t)Np + 1), hs) == cudaSuccess &&
         dev_memset(row + Np, 0, sizeof(int32_t), hs) == cudaSuccess &&
         sssp_rows(plan, row, Np, Np, 0, 1, nullptr, hs) == EAR_OK;
    if (on) {
      EAR_LAUNCH(k_row_far, grid_for(n_real), 256, 0, hs)(row, n_real, row + Np);
      on = readback_direct(host(), row + Np, sizeof(int32_t), hs) == cudaSuccess &&
           cudaEventRecord(ev, hs) == cudaSuccess;
    }
    if (!on) cudaGetLastError();
  }
  bool hopeless() { return on && cudaEventSynchronize(ev) == cudaSuccess && *host() >= (int32_t)C16; }
  void finish() {
    if (!hs) return;
    cudaStreamSynchronize(hs);
    if (row) cudaFreeAsync(row, hs);
    cudaStreamSynchronize(hs);
    cudaStreamDestroy(hs);
    if (ev) cudaEventDestroy(ev);
    hs = nullptr;
  }
  ~Precheck() { finish(); }
};

// The packed 16-bit FW on a copy of D (see C16 above).  *done = false (D untouched) when a connected
// pair reached the cap; the caller then runs the int32 FW.  Synchronises the stream once (the check).
//
// Lookahead: round k's phase 3 is split into the tiles of row/column k+1 (MODE_CROSS, first) and the
// rest (MODE_REST).  As soon as the cross tiles are done, round k+1's pivot work -- phase 1 on tile
// (k+1, k+1), the duplicated pivot row Pd, phase 2 on row k+1 -- runs on a side stream while the rest
// of round k proceeds on the main stream (its launch leaves a few CTA slots free for it); round k+1's
// phase 3 waits for both.  The two streams touch disjoint tiles (the rest skips rows/columns k, k+1)
// and alternate between two Pd buffers, so the serial phases 1-2 leave the critical path.
ear_status_t fw_single16(int32_t *D, int64_t ldd, int32_t Np, const int32_t *lab, int32_t n_real, bool *done,
                         cudaStream_t st, ear_plan_s *plan) {
  *done = false;
  if (!g_num_sms) {
    int dev = 0;
    EAR_CUDA_TRY(cudaGetDevice(&dev));
    EAR_CUDA_TRY(cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev));
  }
  cudaStream_t side;
  cudaEvent_t ev_cross, ev_pivot;
  EAR_TRY(side_stream(&side, &ev_cross, &ev_pivot));
  const bool lookahead = env_int("EAR_FW16_LOOKAHEAD", 1) != 0;
  const int nt = Np / TILE;
  const double tile_ops = (double)TILE * TILE * TILE;
  uint16_t *D16 = nullptr;
  uint32_t *Pd = nullptr;   // two 128 x Np buffers (round parity)
  int32_t *bad = nullptr;
  if (cudaMallocAsync((void **)&D16, sizeof(uint16_t) * (size_t)Np * Np, st) != cudaSuccess ||
      cudaMallocAsync((void **)&Pd, 2 * sizeof(uint32_t) * (size_t)TILE * Np, st) != cudaSuccess ||
      cudaMallocAsync((void **)&bad, sizeof(int32_t), st) != cudaSuccess) {
    cudaGetLastError();
    if (D16) cudaFreeAsync(D16, st);
    if (Pd) cudaFreeAsync(Pd, st);
    return EAR_OK;   // no room for the 16-bit copy: the int32 path runs
  }
  const int KC = fw16_kc();
  ear_status_t s = EAR_OK;
  CUtensorMap mA, mB[2];
  s = make_map_t(&mA, CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, D16, Np, Np, Np, KC);
  for (int b = 0; b < 2 && s == EAR_OK; ++b)
    s = make_map_t(&mB[b], CU_TENSOR_MAP_DATA_TYPE_UINT32, 4, Pd + (size_t)b * TILE * Np, TILE, Np, Np, KC);
  const int64_t ndup = (int64_t)TILE * (Np / 4);
  if (s == EAR_OK) {
    int sc = prof_begin(PK_FW16_CONV, st);
    EAR_LAUNCH(k_to16, grid_for((int64_t)Np * (Np / 4)), 256, 0, st)(D, ldd, D16, Np);
    prof_end(sc, st, 0);
  }
  // phases 1 and 2 of round k on stream q (Pd buffer k & 1)
  auto pivot = [&](int k, cudaStream_t q) -> ear_status_t {
    uint16_t *P16 = D16 + (int64_t)k * TILE * Np;
    uint32_t *Pk = Pd + (size_t)(k & 1) * TILE * Np;
    const bool on_side = q != st;   // lookahead: overlapped with phase 3, reported apart
    int s1 = prof_begin(on_side ? PK_FW_SIDE_P1 : PK_FW_P1, q);
    EAR_LAUNCH(k_fw_phase1_16, 1, NT, 0, q)(P16 + (int64_t)k * TILE, Np);
    prof_end(s1, q, tile_ops);
    int s2 = prof_begin(on_side ? PK_FW_SIDE_P2 : PK_FW_P2, q);
    EAR_LAUNCH(k_dup16, grid_for(ndup), 256, 0, q)(P16, Np, Pk);   // B of phase 2: the pre-phase-2 row
    TileJob16 J{D16, Np, k * TILE, k, nt, MODE_PIVOT_ROW, 1, 0};
    EAR_TRY(launch16<Fw16Tile>(mA, mB[k & 1], J, nt - 1, q));
    EAR_LAUNCH(k_dup16, grid_for(ndup), 256, 0, q)(P16, Np, Pk);   // B of phase 3
    prof_end(s2, q, (nt - 1) * tile_ops);
    return EAR_OK;
  };
  if (s == EAR_OK && nt > 0) s = pivot(0, st);
  // Cap precheck, overlapped with rounds 0-3: the exact distance row of reduced vertex 0 by one
  // single-source SSSP on a helper stream.  Its eccentricity is a lower bound on the largest finite
  // distance; when it already reaches the cap, a connected pair is capped for sure, so the packed FW
  // is abandoned after round 3 instead of running to the end and being thrown away (cfg5: diameter
  // ~42.8k).  Vertex 0 sits at a corner of the spatially coherent labellings, so its eccentricity is
  // close to the diameter.  Only with a plan (plain FW, re-reduced pieces) and a large FW.
  Precheck pc;
  if (s == EAR_OK) pc.start(plan, Np, n_real, nt);
  bool hopeless = false;
  for (int k = 0; k < nt && s == EAR_OK; ++k) {
    if (k == 4 && pc.hopeless()) {   // rounds 0-3 (~4 ms at cfg4 sizes) cover the SSSP: the host rarely waits
      hopeless = true;
      break;
    }
    TileJob16 J{D16, Np, k * TILE, k, nt, MODE_UPPER, 1, 0};
    const int64_t nup = (int64_t)(nt - 1) * nt / 2;
    if (!lookahead || k + 1 == nt) {
      int s3 = prof_begin(PK_FW_P3_16, st);
      s = launch16<Fw16Tile>(mA, mB[k & 1], J, nup, st);
      prof_end(s3, st, nup * tile_ops);
      if (s == EAR_OK && k + 1 < nt) s = pivot(k + 1, st);
      continue;
    }
    int s3 = prof_begin(PK_FW_P3_16, st);
    J.mode = MODE_CROSS;
    s = launch16<Fw16Tile>(mA, mB[k & 1], J, nt - 1, st);
    prof_end(s3, st, (nt - 1) * tile_ops);
    if (s != EAR_OK) break;
    cudaError_t e = cudaEventRecord(ev_cross, st);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(side, ev_cross, 0);
    if (e != cudaSuccess) { set_error("fw_single16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; break; }
    s = pivot(k + 1, side);
    if (s != EAR_OK) break;
    e = cudaEventRecord(ev_pivot, side);
    if (e != cudaSuccess) { set_error("fw_single16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; break; }
    J.mode = MODE_REST;
    const int64_t nrest = (int64_t)(nt - 2) * (nt - 1) / 2;
    int s4 = prof_begin(PK_FW_P3_16, st);
    s = launch16<Fw16Tile>(mA, mB[k & 1], J, nrest, st, lookahead_reserve(nrest, nt - 1));
    prof_end(s4, st, nrest * tile_ops);
    if (s == EAR_OK) {
      e = cudaStreamWaitEvent(st, ev_pivot, 0);
      if (e != cudaSuccess) { set_error("fw_single16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
    }
  }
  if (s != EAR_OK) cudaStreamWaitEvent(st, ev_pivot, 0);   // never leave side work behind the frees
  pc.finish();
  int32_t h_bad = 1;
  if (s == EAR_OK && hopeless) prof_fw16_precheck();
  if (s == EAR_OK && !hopeless) {
    int sc = prof_begin(PK_FW16_CONV, st);
    dev_memset(bad, 0, sizeof(int32_t), st);
    EAR_LAUNCH(k_check16, grid_for((int64_t)Np * (Np / 8)), 256, 0, st)(D16, Np, lab, n_real, bad);
    prof_end(sc, st, 0);
    Readback rb(st);
    cudaError_t e = rb.get(&h_bad, bad, sizeof(int32_t));
    if (e == cudaSuccess) e = rb.sync();
    if (e != cudaSuccess) { set_error("fw_single16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  }
  if (s == EAR_OK && h_bad == 0) {
    int sc = prof_begin(PK_FW16_CONV, st);
    EAR_LAUNCH(k_from16, grid_for((int64_t)Np * (Np / 4)), 256, 0, st)(D16, Np, D, ldd);
    prof_end(sc, st, 0);
    *done = true;
  }
  cudaFreeAsync(D16, st);
  cudaFreeAsync(Pd, st);
  cudaFreeAsync(bad, st);
  if (s != EAR_OK) return s;
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

}  // namespace

ear_status_t fw_init_D(const ear_plan_s *plan, int32_t *D, int64_t ldd, int32_t Np, int32_t row0, int32_t rows,
                       cudaStream_t st) {
  int64_t total = (int64_t)rows * (Np / 4);
  int grid = (int)std::min<int64_t>(ceil_div(total, 256), 148 * 32);
  int s0 = prof_begin(PK_FW_INIT, st);
  if (total > 0) EAR_LAUNCH(k_init_D, grid, 256, 0, st)(D, ldd, Np, row0, rows);
  if (plan->n_redges > 0) {
    int g2 = (int)std::min<int64_t>(ceil_div(plan->n_redges, 256), 148 * 32);
    EAR_LAUNCH(k_init_edges, g2, 256, 0, st)(plan->re_u, plan->re_v, plan->re_w, plan->n_redges, D, ldd, row0, rows);
  }
  prof_end(s0, st, 0);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// Single GPU: full symmetric D (Np x Np).  With allow16 the packed 16-bit FW runs first on a copy and
// its result is kept when no connected pair (labels lab over [0, n_real), or one component when lab is
// NULL) reached the 16-bit cap; otherwise, or without allow16, the int32 FW below runs.
ear_status_t fw_single(int32_t *D, int64_t ldd, int32_t Np, cudaStream_t st, const int32_t *lab, int32_t n_real,
                       bool allow16, ear_plan_s *plan) {
  if (allow16 && Np >= 2 * TILE) {
    bool done = false;
    EAR_TRY(fw_single16(D, ldd, Np, lab, n_real, &done, st, plan));
    prof_fw16(done);
    if (done) return EAR_OK;
  }
  const int nt = Np / TILE;
  const double tile_ops = (double)TILE * TILE * TILE;
  CUtensorMap map;
  EAR_TRY(make_map(&map, D, Np, Np, ldd, fw_kc()));
  for (int k = 0; k < nt; ++k) {
    int32_t *Pk = D + (int64_t)k * TILE * ldd;            // pivot row block
    int s1 = prof_begin(PK_FW_P1, st);
    EAR_LAUNCH(k_fw_phase1, 1, NT, 0, st)(Pk + (int64_t)k * TILE, ldd);
    prof_end(s1, st, tile_ops);
    TileJob J{D, ldd, k * TILE, k, nt, 0, nt, MODE_PIVOT_ROW, 1, 0};
    int s2 = prof_begin(PK_FW_P2, st);
    EAR_TRY(launch_tiles(map, J, nt - 1, st));
    prof_end(s2, st, (nt - 1) * tile_ops);
    J.mode = MODE_UPPER;
    const int64_t nup = (int64_t)(nt - 1) * nt / 2;
    int s3 = prof_begin(PK_FW_P3, st);
    EAR_TRY(launch_tiles(map, J, nup, st));
    prof_end(s3, st, nup * tile_ops);
  }
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// ---------------------------------------------------------------------------- row-block sharding
// Symmetric row-block sharding.  Tile rows are dealt to ranks in a zig-zag (rows r and 2P-1-r of every
// group of 2P), so the UPPER tiles (ti, tj >= ti) -- the only authoritative ones -- balance across
// ranks; rank r stores its owned tile rows (ascending) as 128-row blocks.  Round k:
//   1. every rank writes its pieces of the pivot row block into prow (tile (k, j >= k) from the owner
//      of row k, tiles (i < k, k) transposed from the owners of rows i), INF elsewhere, and an
//      all-reduce(MIN) over NCCL assembles the block on every rank;
//   2. every rank closes the pivot tile (phase 1) and updates the pivot row block (phase 2) locally;
//   3. owners copy the updated pivot pieces back into their storage;
//   4. every rank updates its owned upper tiles outside row/column k (phase 3), both operands from prow.
// Per-rank min-plus work is (N_r^3 / 2) / P + the redundant phase 1/2, i.e. the single-GPU symmetric
// halving survives the sharding.  The final D is assembled by scattering every rank's upper tiles and
// their mirrors into an INF-filled full matrix and one all-reduce(MIN).

std::vector<int32_t> shard_rows(int32_t nt, int32_t P, int32_t rank) {
  std::vector<int32_t> rows;
  for (int32_t ti = 0; ti < nt; ++ti) {
    const int32_t o = ti % (2 * P);
    if ((o < P ? o : 2 * P - 1 - o) == rank) rows.push_back(ti);
  }
  return rows;
}

struct Shard {
  int32_t *S = nullptr;        // owned storage: nown x 128 rows x ldd
  int64_t ldd = 0;
  int32_t Np = 0, nt = 0, P = 1, rank = 0, nown = 0;
  std::vector<int32_t> rows;
  int32_t *d_rows = nullptr;
  int64_t *d_pre = nullptr;
};

static ear_status_t shard_setup(Shard *sh, int32_t *S, int64_t ldd, int32_t Np, int32_t P, int32_t rank,
                                cudaStream_t st) {
  sh->S = S; sh->ldd = ldd; sh->Np = Np; sh->nt = Np / TILE; sh->P = P; sh->rank = rank;
  sh->rows = shard_rows(sh->nt, P, rank);
  sh->nown = (int32_t)sh->rows.size();
  std::vector<int64_t> pre(sh->nown + 1, 0);
  for (int32_t r = 0; r < sh->nown; ++r) pre[r + 1] = pre[r] + (sh->nt - sh->rows[r]);
  const size_t nr = std::max<int32_t>(sh->nown, 1);
  EAR_CUDA_TRY(cudaMallocAsync((void **)&sh->d_rows, sizeof(int32_t) * nr, st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&sh->d_pre, sizeof(int64_t) * (nr + 1), st));
  if (sh->nown > 0) {
    EAR_CUDA_TRY(cudaMemcpyAsync(sh->d_rows, sh->rows.data(), sizeof(int32_t) * sh->nown, cudaMemcpyHostToDevice, st));
    EAR_CUDA_TRY(cudaMemcpyAsync(sh->d_pre, pre.data(), sizeof(int64_t) * (sh->nown + 1), cudaMemcpyHostToDevice, st));
    EAR_CUDA_TRY(cudaStreamSynchronize(st));   // host vectors are about to go out of scope
  }
  return EAR_OK;
}

static void shard_free(Shard *sh, cudaStream_t st) {
  if (sh->d_rows) cudaFreeAsync(sh->d_rows, st);
  if (sh->d_pre) cudaFreeAsync(sh->d_pre, st);
  sh->d_rows = nullptr; sh->d_pre = nullptr;
}

static ear_status_t fill(int32_t *p, int64_t n, int32_t v, cudaStream_t st) {
  if (n <= 0) return EAR_OK;
  EAR_LAUNCH(k_fill, (int)std::min<int64_t>(ceil_div(n, 256), 148 * 16), 256, 0, st)(p, n, v);
  return EAR_OK;
}

// this rank's pieces of round k's pivot row block (see k_prow_xfer)
static void shard_pieces(const Shard &sh, int k, int *posk, int *mk) {
  *posk = -1;
  *mk = 0;
  for (int32_t r = 0; r < sh.nown; ++r) {
    if (sh.rows[r] < k) ++*mk;
    if (sh.rows[r] == k) *posk = r;
  }
}

template <class TS, class TP>
static ear_status_t shard_xfer_t(const Shard &sh, TS *S, int64_t ld, int k, TP *prow, int dir, cudaStream_t st) {
  int posk, mk;
  shard_pieces(sh, k, &posk, &mk);
  const int np = (posk >= 0 ? sh.nt - k : 0) + mk;
  if (np == 0) return EAR_OK;
  EAR_LAUNCH((k_prow_xfer<TS, TP>), dim3(16, np), 256, 0, st)(S, ld, sh.d_rows, k, sh.nt, posk, prow, sh.Np, dir);
  return EAR_OK;
}

static ear_status_t shard_xfer(const Shard &sh, int k, int32_t *prow, int dir, cudaStream_t st) {
  return shard_xfer_t<int32_t, int32_t>(sh, sh.S, sh.ldd, k, prow, dir, st);
}

// phases 1 and 2 on the assembled pivot row block
static ear_status_t shard_pivot(int32_t *prow, const CUtensorMap &map_prow, int32_t Np, int k, cudaStream_t st) {
  const int nt = Np / TILE;
  const double tile_ops = (double)TILE * TILE * TILE;
  int s1 = prof_begin(PK_FW_P1, st);
  EAR_LAUNCH(k_fw_phase1, 1, NT, 0, st)(prow + (int64_t)k * TILE, Np);
  prof_end(s1, st, tile_ops);
  TileJob J{prow, Np, 0, k, nt, k, 1, MODE_PIVOT_ROW, 0, 0, nullptr, nullptr, 0, 0, -1};
  int s2 = prof_begin(PK_FW_P2, st);
  EAR_TRY(launch_tiles(map_prow, J, nt - 1, st));
  prof_end(s2, st, (nt - 1) * tile_ops);
  return EAR_OK;
}

static ear_status_t shard_phase3(const Shard &sh, const CUtensorMap &map_prow, int k, cudaStream_t st) {
  int mk = 0, posk = -1;
  for (int32_t r = 0; r < sh.nown; ++r) {
    if (sh.rows[r] < k) ++mk;
    if (sh.rows[r] == k) posk = r;
  }
  int64_t total = 0;
  for (int32_t r = 0; r < sh.nown; ++r) {
    const int32_t ti = sh.rows[r];
    total += ti == k ? 0 : (sh.nt - ti) - (ti < k ? 1 : 0);
  }
  TileJob J{sh.S, sh.ldd, 0, k, sh.nt, 0, sh.nown, MODE_LIST, 0, 0, sh.d_rows, sh.d_pre, sh.nown, mk, posk};
  int s3 = prof_begin(PK_FW_P3, st);
  EAR_TRY(launch_tiles(map_prow, J, total, st));
  prof_end(s3, st, (double)total * TILE * TILE * TILE);
  return EAR_OK;
}

ear_status_t fw_sharded(int32_t *S, int64_t ldd, int32_t Np, ear_comm_s *comm, cudaStream_t st) {
  Shard sh;
  EAR_TRY(shard_setup(&sh, S, ldd, Np, comm->nranks, comm->rank, st));
  int32_t *prow = nullptr;
  EAR_CUDA_TRY(cudaMallocAsync((void **)&prow, sizeof(int32_t) * (size_t)TILE * Np, st));
  CUtensorMap map_prow;
  ear_status_t status = make_map(&map_prow, prow, TILE, Np, Np, fw_kc());
  for (int k = 0; k < sh.nt && status == EAR_OK; ++k) {
    status = fill(prow, (int64_t)TILE * Np, INF, st);
    if (status == EAR_OK) status = shard_xfer(sh, k, prow, 0, st);
    if (status == EAR_OK) {
      int sc = prof_begin(PK_COMM, st);
      status = comm_allreduce_min(comm, prow, (int64_t)TILE * Np, st);
      prof_end(sc, st, 0);
    }
    if (status == EAR_OK) status = shard_pivot(prow, map_prow, Np, k, st);
    if (status == EAR_OK) status = shard_xfer(sh, k, prow, 1, st);
    if (status == EAR_OK) status = shard_phase3(sh, map_prow, k, st);
  }
  cudaFreeAsync(prow, st);
  shard_free(&sh, st);
  if (status != EAR_OK) return status;
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// ---------------------------------------------------------------- 16-bit row-block sharding
// The sharded schedule above on packed 16-bit owned rows (the cap C16 and its exactness argument are
// those of fw_single16).  The exchange stays int32 -- NCCL has no 16-bit MIN: the owned u16 pieces are
// widened into the INF-filled int32 pivot row block and all-reduced; the block is narrowed back to u16
// (values <= C16, so exactly the capped values) and closed by the packed phases 1-2 of fw_single16's
// pivot() -- phase 1 on the pivot tile, phase 2 as one product against the duplicated pre-phase-2 row --
// then scattered back to the owners; its duplicated copy is the B operand of the packed phase-3
// kernel, which updates the owned u16 rows (MODE_LIST).
// comm == nullptr: the shards are virtual ranks on this device sharing the block (their pieces are
// disjoint, so no exchange is needed).  The range check runs over every rank's owned upper tiles and
// is MIN-reduced; *done = false leaves the int32 owned storage untouched for the int32 schedule.
static ear_status_t phase3_16(const Shard &sh, uint16_t *S16, const CUtensorMap &mA, const CUtensorMap &mB, int k,
                              int mode, cudaStream_t st, int reserve = 0) {   // reserve < 0: lookahead_reserve
  int mk = 0, posk = -1, posk1 = -1;
  int64_t total = 0;
  for (int32_t r = 0; r < sh.nown; ++r) {
    const int32_t ti = sh.rows[r];
    if (ti < k) ++mk;
    if (ti == k) posk = r;
    if (ti == k + 1) posk1 = r;
  }
  for (int32_t r = 0; r < sh.nown; ++r) {
    const int32_t ti = sh.rows[r];
    const int64_t all = ti == k ? 0 : (sh.nt - ti) - (ti < k ? 1 : 0);
    const int64_t cross = (ti == k + 1 ? sh.nt - ti : 0) + (ti < k ? 1 : 0);
    total += mode == MODE_LIST ? all : mode == MODE_LIST_CROSS ? cross : all - cross;
  }
  if (total == 0) return EAR_OK;
  if (reserve < 0) reserve = lookahead_reserve(total, (sh.nt - 1 + sh.P - 1) / sh.P);   // owner-side phase 2
  TileJob16 J{S16, sh.Np, 0, k, sh.nt, mode, 0, 0, sh.d_rows, sh.d_pre, sh.nown, mk, posk};
  J.posk1 = posk1;
  int s3 = prof_begin(PK_FW_P3_16, st);
  EAR_TRY(launch16<Fw16Tile>(mA, mB, J, total, st, reserve));
  prof_end(s3, st, (double)total * TILE * TILE * TILE);
  return EAR_OK;
}

// Lookahead (as fw_single16's): round k's phase 3 is split into the owned tiles of row/column k+1
// (MODE_LIST_CROSS, first) and the rest (MODE_LIST_REST); once the cross tiles are done, round k+1's
// pivot chain -- pieces into the exchange block, the all-reduce, narrowing, phases 1-2, scatter back --
// runs on the side stream (NCCL included) while the rest of round k proceeds; the two touch disjoint
// tiles, the narrowed block and its duplicate alternate between two buffers by round parity, and round
// k+1's phase 3 waits for the chain.
static ear_status_t fw_sharded16(std::vector<Shard *> &sh, int32_t Np, ear_comm_s *comm, const int32_t *lab,
                                 int32_t n_real, bool *done, cudaStream_t st, bool timing_only = false,
                                 ear_plan_s *plan = nullptr) {
  *done = false;
  const int nt = Np / TILE;
  if (nt < 2) return EAR_OK;
  if (!g_num_sms) {
    int dev = 0;
    EAR_CUDA_TRY(cudaGetDevice(&dev));
    EAR_CUDA_TRY(cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev));
  }
  cudaStream_t side;
  cudaEvent_t ev_cross, ev_pivot;
  EAR_TRY(side_stream(&side, &ev_cross, &ev_pivot));
  const bool lookahead = env_int("EAR_FW16_LOOKAHEAD", 1) != 0;
  const size_t R = sh.size();
  std::vector<uint16_t *> S16(R, nullptr);
  int32_t *prow = nullptr, *flag = nullptr;
  uint16_t *p16 = nullptr;   // two 128 x Np buffers (round parity), as Pd
  uint32_t *Pd = nullptr;
  uint16_t *L16 = nullptr, *ptile = nullptr;   // this rank's pivot-row pieces; the broadcast pivot tile
  uint32_t *Ld = nullptr;                      // L16 duplicated (phase-2 B operand)
  const int P = comm ? comm->nranks : (int)sh.size();
  bool ok = cudaMallocAsync((void **)&prow, sizeof(int32_t) * (size_t)TILE * Np, st) == cudaSuccess &&
            cudaMallocAsync((void **)&L16, sizeof(uint16_t) * (size_t)TILE * Np, st) == cudaSuccess &&
            cudaMallocAsync((void **)&Ld, sizeof(uint32_t) * (size_t)TILE * Np, st) == cudaSuccess &&
            cudaMallocAsync((void **)&ptile, sizeof(uint16_t) * TILE * TILE, st) == cudaSuccess &&
            cudaMallocAsync((void **)&p16, 2 * sizeof(uint16_t) * (size_t)TILE * Np, st) == cudaSuccess &&
            cudaMallocAsync((void **)&Pd, 2 * sizeof(uint32_t) * (size_t)TILE * Np, st) == cudaSuccess &&
            cudaMallocAsync((void **)&flag, sizeof(int32_t), st) == cudaSuccess;
  for (size_t r = 0; r < R && ok; ++r)
    ok = cudaMallocAsync((void **)&S16[r], sizeof(uint16_t) * (size_t)std::max(sh[r]->nown, 1) * TILE * Np, st) ==
         cudaSuccess;
  auto release = [&]() {
    for (size_t r = 0; r < R; ++r)
      if (S16[r]) cudaFreeAsync(S16[r], st);
    if (prow) cudaFreeAsync(prow, st);
    if (p16) cudaFreeAsync(p16, st);
    if (Pd) cudaFreeAsync(Pd, st);
    if (L16) cudaFreeAsync(L16, st);
    if (Ld) cudaFreeAsync(Ld, st);
    if (ptile) cudaFreeAsync(ptile, st);
    if (flag) cudaFreeAsync(flag, st);
  };
  if (!ok) {   // no room for the 16-bit copies: the int32 schedule runs
    cudaGetLastError();
    release();
    return EAR_OK;
  }
  const int KC = fw16_kc();
  const int64_t nblk = (int64_t)TILE * Np;
  CUtensorMap mA[2], mB[2], mL, mLd;
  ear_status_t s = make_map_t(&mL, CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, L16, TILE, Np, Np, KC);
  if (s == EAR_OK) s = make_map_t(&mLd, CU_TENSOR_MAP_DATA_TYPE_UINT32, 4, Ld, TILE, Np, Np, KC);
  for (int b = 0; b < 2 && s == EAR_OK; ++b) {
    s = make_map_t(&mA[b], CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, p16 + b * nblk, TILE, Np, Np, KC);
    if (s == EAR_OK) s = make_map_t(&mB[b], CU_TENSOR_MAP_DATA_TYPE_UINT32, 4, Pd + b * nblk, TILE, Np, Np, KC);
  }
  if (s == EAR_OK) {
    int sc = prof_begin(PK_FW16_CONV, st);
    for (size_t r = 0; r < R; ++r)
      if (sh[r]->nown > 0)
        EAR_LAUNCH(k_to16r, grid_for((int64_t)sh[r]->nown * TILE * (Np / 4)), 256, 0, st)(
            sh[r]->S, sh[r]->ldd, S16[r], Np, (int64_t)sh[r]->nown * TILE, Np);
    prof_end(sc, st, 0);
  }
  // round k's pivot chain on stream q, with the phase 2 done by the owners of the pieces:
  //   every rank copies its pieces of the pivot row block into L (u16, C16 elsewhere -- above every
  //   capped value, so the MIN exchange ignores it); the owner of row k closes the pivot tile in L
  //   (phase 1) and broadcasts it (32 KB); every rank applies phase 2 to ITS pieces only (MODE_PIECES,
  //   B = L duplicated before phase 2, as fw_single16's single-product phase 2); the pieces are
  //   widened and all-reduced (MIN) into the full phase-2-complete block, which is narrowed into the
  //   A operand of phase 3 (buffer k & 1), duplicated into its B operand and scattered back to the
  //   owners.  No phase 2 is computed twice: each tile of the pivot row is updated by its contributor.
  auto chain = [&](int k, cudaStream_t q) -> ear_status_t {
    const bool on_side = q != st;
    uint16_t *P16 = p16 + (k & 1) * nblk;
    uint32_t *Pk = Pd + (k & 1) * nblk;
    EAR_LAUNCH(k_fill16, grid_for(nblk / 2), 256, 0, q)(L16, nblk / 2, (uint32_t)C16 * 0x10001u);
    for (size_t r = 0; r < R; ++r)
      if (sh[r]->nown > 0) EAR_TRY((shard_xfer_t<uint16_t, uint16_t>(*sh[r], S16[r], Np, k, L16, 0, q)));
    const int o = k % (2 * P), owner = o < P ? o : 2 * P - 1 - o;
    const bool mine = comm ? comm->rank == owner : true;   // emulated: some shard owns it
    int s1 = prof_begin(on_side ? PK_FW_SIDE_P1 : PK_FW_P1, q);
    if (mine) EAR_LAUNCH(k_fw_phase1_16, 1, NT, 0, q)(L16 + (int64_t)k * TILE, Np);
    prof_end(s1, q, mine ? (double)TILE * TILE * TILE : 0.0);
    if (comm && P > 1) {   // the closed pivot tile from its owner
      int sc = prof_begin(PK_COMM, q);
      const size_t pitch = sizeof(uint16_t) * Np, w = sizeof(uint16_t) * TILE;
      if (mine) EAR_CUDA_TRY(cudaMemcpy2DAsync(ptile, w, L16 + (int64_t)k * TILE, pitch, w, TILE, cudaMemcpyDeviceToDevice, q));
      EAR_TRY(comm_bcast(comm, reinterpret_cast<int32_t *>(ptile), TILE * TILE / 2, owner, q));
      if (!mine) EAR_CUDA_TRY(cudaMemcpy2DAsync(L16 + (int64_t)k * TILE, pitch, ptile, w, w, TILE, cudaMemcpyDeviceToDevice, q));
      prof_end(sc, q, 0);
    }
    int s2 = prof_begin(on_side ? PK_FW_SIDE_P2 : PK_FW_P2, q);
    EAR_LAUNCH(k_dup16, grid_for(nblk / 4), 256, 0, q)(L16, Np, Ld);
    double p2 = 0;
    for (size_t r = 0; r < R; ++r) {
      int posk, mk;
      shard_pieces(*sh[r], k, &posk, &mk);
      const int64_t n2 = mk + (posk >= 0 ? nt - 1 - k : 0);
      if (n2 == 0) continue;
      TileJob16 J2{L16, Np, 0, k, nt, MODE_PIECES, 0, 0, sh[r]->d_rows, sh[r]->d_pre, sh[r]->nown, mk, posk};
      EAR_TRY(launch16<Fw16Tile>(mL, mLd, J2, n2, q));
      p2 += (double)n2 * TILE * TILE * TILE;
    }
    prof_end(s2, q, p2);
    EAR_LAUNCH(k_widen16, grid_for(nblk / 4), 256, 0, q)(L16, prow, nblk);
    if (comm) {
      int sc = prof_begin(PK_COMM, q);
      EAR_TRY(comm_allreduce_min(comm, prow, nblk, q));
      prof_end(sc, q, 0);
    }
    EAR_LAUNCH(k_prow_to16, grid_for(nblk / 4), 256, 0, q)(prow, P16, Pk, nblk);
    for (size_t r = 0; r < R; ++r)
      if (sh[r]->nown > 0) EAR_TRY((shard_xfer_t<uint16_t, uint16_t>(*sh[r], S16[r], Np, k, P16, 1, q)));
    return EAR_OK;
  };
  if (s == EAR_OK) s = chain(0, st);
  Precheck pc;   // as fw_single16's; every rank decides the same
  if (s == EAR_OK && !timing_only) pc.start(plan, Np, n_real, nt);
  bool hopeless = false;
  for (int k = 0; k < nt && s == EAR_OK; ++k) {
    if (k == 4 && pc.hopeless()) {
      hopeless = true;
      break;
    }
    const CUtensorMap &A = mA[k & 1], &B = mB[k & 1];
    if (!lookahead || k + 1 == nt) {
      for (size_t r = 0; r < R && s == EAR_OK; ++r) s = phase3_16(*sh[r], S16[r], A, B, k, MODE_LIST, st);
      if (s == EAR_OK && k + 1 < nt) s = chain(k + 1, st);
      continue;
    }
    for (size_t r = 0; r < R && s == EAR_OK; ++r) s = phase3_16(*sh[r], S16[r], A, B, k, MODE_LIST_CROSS, st);
    if (s != EAR_OK) break;
    cudaError_t e = cudaEventRecord(ev_cross, st);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(side, ev_cross, 0);
    if (e != cudaSuccess) { set_error("fw_sharded16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; break; }
    s = chain(k + 1, side);
    e = cudaEventRecord(ev_pivot, side);   // recorded even after an error: the main stream waits for it
    if (s == EAR_OK && e != cudaSuccess) { set_error("fw_sharded16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
    for (size_t r = 0; r < R && s == EAR_OK; ++r)
      s = phase3_16(*sh[r], S16[r], A, B, k, MODE_LIST_REST, st, -1);
    e = cudaStreamWaitEvent(st, ev_pivot, 0);
    if (s == EAR_OK && e != cudaSuccess) { set_error("fw_sharded16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  }
  pc.finish();
  if (s == EAR_OK && hopeless) {   // the int32 schedule runs on the untouched int32 rows
    prof_fw16_precheck();
    release();
    EAR_CUDA_TRY(cudaGetLastError());
    return EAR_OK;
  }
  int32_t h_flag = -1;
  if (s == EAR_OK && timing_only) {   // apsp_reduced_rank_timing: no check, no result
    release();
    EAR_CUDA_TRY(cudaGetLastError());
    return EAR_OK;
  }
  if (s == EAR_OK) {
    int sc = prof_begin(PK_FW16_CONV, st);
    dev_memset(flag, 0, sizeof(int32_t), st);
    for (size_t r = 0; r < R; ++r)
      if (sh[r]->nown > 0)
        EAR_LAUNCH(k_check16_list, grid_for((int64_t)sh[r]->nown * TILE * (Np / 8)), 256, 0, st)(
            S16[r], Np, sh[r]->d_rows, sh[r]->nown, Np, lab, n_real, flag);
    prof_end(sc, st, 0);
    if (comm) s = comm_allreduce_min(comm, flag, 1, st);
    Readback rb(st);
    cudaError_t e = rb.get(&h_flag, flag, sizeof(int32_t));
    if (e == cudaSuccess) e = rb.sync();
    if (s == EAR_OK && e != cudaSuccess) { set_error("fw_sharded16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  }
  if (s == EAR_OK && h_flag == 0) {
    int sc = prof_begin(PK_FW16_CONV, st);
    for (size_t r = 0; r < R; ++r)
      if (sh[r]->nown > 0)
        EAR_LAUNCH(k_from16r, grid_for((int64_t)sh[r]->nown * TILE * (Np / 4)), 256, 0, st)(
            S16[r], Np, sh[r]->S, sh[r]->ldd, (int64_t)sh[r]->nown * TILE, Np);
    prof_end(sc, st, 0);
    *done = true;
  }
  release();
  if (s != EAR_OK) return s;
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// Sharded FW on a rank's owned int32 rows: the 16-bit schedule first (allow16), the int32 one when it
// did not apply.  lab / n_real as for fw_single.
ear_status_t fw_sharded_auto(int32_t *S, int64_t ldd, int32_t Np, ear_comm_s *comm, const int32_t *lab,
                             int32_t n_real, bool allow16, cudaStream_t st, ear_plan_s *plan) {
  if (allow16 && Np >= 2 * TILE) {
    Shard sh;
    EAR_TRY(shard_setup(&sh, S, ldd, Np, comm->nranks, comm->rank, st));
    std::vector<Shard *> v{&sh};
    bool done = false;
    ear_status_t s = fw_sharded16(v, Np, comm, lab, n_real, &done, st, false, plan);
    shard_free(&sh, st);
    EAR_TRY(s);
    prof_fw16(done);
    if (done) return EAR_OK;
  }
  return fw_sharded(S, ldd, Np, comm, st);
}

// One rank's device work of a P-rank packed sharded FW, without the other ranks and the exchange
// (apsp_reduced_rank_timing: per-rank compute scaling measured on one GPU).
ear_status_t fw_rank_timing(const ear_plan_s *plan, int32_t Np, int32_t P, int32_t rank, cudaStream_t st) {
  const size_t nown = shard_rows(Np / TILE, P, rank).size();
  int32_t *S = nullptr;
  EAR_CUDA_TRY(cudaMallocAsync((void **)&S, sizeof(int32_t) * std::max<size_t>(nown, 1) * TILE * Np, st));
  Shard sh;
  ear_status_t s = shard_setup(&sh, S, Np, Np, P, rank, st);
  for (int32_t lr = 0; lr < sh.nown && s == EAR_OK; ++lr)
    s = fw_init_D(plan, S + (int64_t)lr * TILE * Np, Np, Np, sh.rows[lr] * TILE, TILE, st);
  bool done = false;
  std::vector<Shard *> v{&sh};
  if (s == EAR_OK) s = fw_sharded16(v, Np, nullptr, nullptr, plan->n_reduced, &done, st, true);
  shard_free(&sh, st);
  cudaFreeAsync(S, st);
  return s;
}

// Full D from every rank's owned upper tiles (INF fill + scatter + all-reduce MIN).
ear_status_t fw_sharded_gather(const int32_t *S, int64_t ldd, int32_t Np, int32_t *Df, int64_t ldf, ear_comm_s *comm,
                               cudaStream_t st) {
  Shard sh;
  EAR_TRY(shard_setup(&sh, const_cast<int32_t *>(S), ldd, Np, comm->nranks, comm->rank, st));
  ear_status_t status = EAR_OK;
  if (ldf == Np) {
    status = fill(Df, (int64_t)Np * Np, INF, st);
  } else {
    for (int32_t r = 0; r < Np && status == EAR_OK; ++r) status = fill(Df + (int64_t)r * ldf, Np, INF, st);
  }
  if (status == EAR_OK && sh.nown > 0) {
    dim3 g(16, sh.nt, sh.nown);
    EAR_LAUNCH(k_scatter_upper, g, 256, 0, st)(sh.S, sh.ldd, sh.d_rows, Df, ldf);
  }
  if (status == EAR_OK) {
    int sc = prof_begin(PK_COMM, st);
    if (ldf == Np) {
      status = comm_allreduce_min(comm, Df, (int64_t)Np * Np, st);
    } else {
      for (int32_t r = 0; r < Np && status == EAR_OK; ++r) status = comm_allreduce_min(comm, Df + (int64_t)r * ldf, Np, st);
    }
    prof_end(sc, st, 0);
  }
  shard_free(&sh, st);
  if (status != EAR_OK) return status;
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

int32_t shard_nown(int32_t nt, int32_t P, int32_t rank) { return (int32_t)shard_rows(nt, P, rank).size(); }

ear_status_t shard_rows_device(int32_t nt, int32_t P, int32_t rank, int32_t **d_rows, int32_t *nown, cudaStream_t st) {
  std::vector<int32_t> rows = shard_rows(nt, P, rank);
  *nown = (int32_t)rows.size();
  EAR_CUDA_TRY(cudaMallocAsync((void **)d_rows, sizeof(int32_t) * std::max<size_t>(rows.size(), 1), st));
  if (!rows.empty()) {
    EAR_CUDA_TRY(cudaMemcpyAsync(*d_rows, rows.data(), sizeof(int32_t) * rows.size(), cudaMemcpyHostToDevice, st));
    EAR_CUDA_TRY(cudaStreamSynchronize(st));
  }
  return EAR_OK;
}

// The same schedule for P ranks emulated in one process on one device (tests of the multi-GPU path on
// one GPU): every virtual rank has its own owned storage, the shared prow stands in for the
// all-reduce (the ranks' pieces are disjoint), and the ranks' upper tiles are scattered into D.
ear_status_t fw_sharded_emulated(ear_plan_s *plan, int32_t *D, int64_t ldd, int32_t Np, int32_t P,
                                 cudaStream_t st) {
  const int nt = Np / TILE;
  std::vector<Shard> sh(P);
  ear_status_t status = EAR_OK;
  for (int r = 0; r < P && status == EAR_OK; ++r) {
    const size_t nown = shard_rows(nt, P, r).size();
    int32_t *S = nullptr;
    EAR_CUDA_TRY(cudaMallocAsync((void **)&S, sizeof(int32_t) * std::max<size_t>(nown, 1) * TILE * Np, st));
    status = shard_setup(&sh[r], S, Np, Np, P, r, st);
    for (int32_t lr = 0; lr < sh[r].nown && status == EAR_OK; ++lr)
      status = fw_init_D(plan, S + (int64_t)lr * TILE * Np, Np, Np, sh[r].rows[lr] * TILE, TILE, st);
  }
  bool done16 = false;
  if (status == EAR_OK && !(plan->flags & EAR_FLAG_FW32) && Np >= 2 * TILE) {
    const int32_t *lab = nullptr;
    status = reduced_labels(plan, Np, st, &lab);
    std::vector<Shard *> v;
    for (int r = 0; r < P; ++r) v.push_back(&sh[r]);
    if (status == EAR_OK) status = fw_sharded16(v, Np, nullptr, lab, plan->n_reduced, &done16, st, false, plan);
    if (status == EAR_OK) prof_fw16(done16);
  }
  int32_t *prow = nullptr;
  if (status == EAR_OK && !done16) {
    cudaError_t e = cudaMallocAsync((void **)&prow, sizeof(int32_t) * (size_t)TILE * Np, st);
    if (e != cudaSuccess) { set_error("emulated prow: %s", cudaGetErrorString(e)); status = EAR_ENOMEM; }
  }
  CUtensorMap map_prow;
  if (status == EAR_OK && !done16) status = make_map(&map_prow, prow, TILE, Np, Np, fw_kc());
  for (int k = 0; k < nt && status == EAR_OK && !done16; ++k) {
    status = fill(prow, (int64_t)TILE * Np, INF, st);
    for (int r = 0; r < P && status == EAR_OK; ++r) status = shard_xfer(sh[r], k, prow, 0, st);
    if (status == EAR_OK) status = shard_pivot(prow, map_prow, Np, k, st);
    for (int r = 0; r < P && status == EAR_OK; ++r) status = shard_xfer(sh[r], k, prow, 1, st);
    for (int r = 0; r < P && status == EAR_OK; ++r) status = shard_phase3(sh[r], map_prow, k, st);
  }
  for (int r = 0; r < P && status == EAR_OK; ++r) {
    if (sh[r].nown == 0) continue;
    dim3 g(16, nt, sh[r].nown);
    EAR_LAUNCH(k_scatter_upper, g, 256, 0, st)(sh[r].S, sh[r].ldd, sh[r].d_rows, D, ldd);
  }
  if (prow) cudaFreeAsync(prow, st);
  for (int r = 0; r < P; ++r) {
    if (sh[r].S) cudaFreeAsync(sh[r].S, st);
    shard_free(&sh[r], st);
  }
  if (status != EAR_OK) return status;
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// connected-component labels of G^r (cached in the plan; padding vertices are their own component)
ear_status_t reduced_labels(ear_plan_s *p, int32_t Np, cudaStream_t st, const int32_t **out) {
  if (!p->cc || p->cc_np != Np) {
    if (p->cc) cudaFreeAsync(p->cc, st);
    p->cc = nullptr;
    int32_t *changed = nullptr;
    EAR_CUDA_TRY(cudaMallocAsync((void **)&p->cc, sizeof(int32_t) * (size_t)Np, st));
    EAR_CUDA_TRY(cudaMallocAsync((void **)&changed, sizeof(int32_t), st));
    p->cc_np = Np;
    EAR_LAUNCH(k_cc_init, grid_for(Np), 256, 0, st)(p->cc, Np);
    ear_status_t s = EAR_OK;
    for (int it = 0; it < 64 && s == EAR_OK; ++it) {
      int32_t h = 0;
      if (p->n_redges == 0) break;
      dev_memset(changed, 0, sizeof(int32_t), st);
      EAR_LAUNCH(k_cc_hook16, grid_for(p->n_redges), 256, 0, st)(p->re_u, p->re_v, p->n_redges, p->cc, changed);
      EAR_LAUNCH(k_cc_jump16, grid_for(Np), 256, 0, st)(p->cc, Np);
      Readback rb(st);
      cudaError_t e = rb.get(&h, changed, sizeof(int32_t));
      if (e == cudaSuccess) e = rb.sync();
      if (e != cudaSuccess) { set_error("reduced_labels: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
      if (!h) break;
    }
    cudaFreeAsync(changed, st);
    EAR_TRY(s);
  }
  *out = p->cc;
  return EAR_OK;
}

}  // namespace ear
