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
enum { MODE_PIVOT_ROW = 0, MODE_UPPER = 1, MODE_LIST = 2 };

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
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, int32_t c0, int32_t c1, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar))
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
  if (J.mode == MODE_UPPER) {
    // upper triangle (a <= b) of the (nt-1) x (nt-1) non-pivot tiles, row-major; row a starts at
    // a*T - a*(a-1)/2
    const int64_t T = J.nt - 1;
    double tt = (double)(2 * T + 1);
    int64_t a = (int64_t)floor((tt - sqrt(tt * tt - 8.0 * (double)idx)) * 0.5);
    if (a < 0) a = 0;
    while (a > 0 && a * T - a * (a - 1) / 2 > idx) --a;
    while ((a + 1) * T - (a + 1) * a / 2 <= idx) ++a;
    const int64_t b = a + (idx - (a * T - a * (a - 1) / 2));
    ti = (int)a < k ? (int)a : (int)a + 1;
    tj = (int)b < k ? (int)b : (int)b + 1;
    lr = ti - J.ti0;
    return;
  }
  // MODE_LIST: the upper tiles (ti, tj >= ti) of the owned rows, without row k and column k.
  // Per round, owned rows ti < k lose tile (ti, k) and row k (if owned) loses all its tiles.
  auto pre = [&](int r) -> int64_t {
    return J.opre[r] - min(r, J.mk) - ((J.posk >= 0 && r > J.posk) ? (int64_t)(J.nt - k) : 0);
  };
  int lo = 0, hi = J.nown - 1;   // largest r with pre(r) <= idx (ties: the last, skipping empty rows)
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (pre(mid) <= idx) lo = mid; else hi = mid - 1;
  }
  lr = lo;
  ti = J.orow[lo];
  tj = ti + (int)(idx - pre(lo));
  if (ti < k && tj >= k) ++tj;
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

// Pivot-row block <-> a rank's owned storage, round k (prow: 128 x Np, leading dimension Np).
//   dir = 0 (gather):  prow[:, ti-block] = S(ti, k)^T for owned ti < k; prow[:, j >= k] = S(k, j) if row k owned
//   dir = 1 (scatter): the inverse, after phases 1 and 2 updated prow
// grid: (16 sub-blocks of 32 x 32, Np/128 column tiles, nown owned rows), 256 threads
__global__ void k_prow_xfer(int32_t *S, int64_t ldd, const int32_t *orow, int32_t k, int32_t *prow, int32_t Np,
                            int dir) {
  __shared__ int32_t t[32][33];
  const int lr = blockIdx.z, ti = orow[lr], tj = blockIdx.y;
  const int bx = blockIdx.x & 3, by = blockIdx.x >> 2;         // 32 x 32 sub-block (bx: x, by: y)
  const int lx = threadIdx.x & 31, ly = threadIdx.x >> 5;      // 32 x 8 threads
  if (ti == k) {               // the pivot row's upper part: plain copy, tiles j >= k
    if (tj < k) return;
    for (int yy = ly; yy < 32; yy += 8) {
      const int64_t row = by * 32 + yy, col = (int64_t)tj * TILE + bx * 32 + lx;
      int32_t *s = S + ((int64_t)lr * TILE + row) * ldd + col;
      int32_t *p = prow + row * Np + col;
      if (dir == 0) *p = *s; else *s = *p;
    }
    return;
  }
  if (ti > k || tj != k) return;   // owned row below the pivot: its tile (ti, k) <-> prow[:, ti-block]^T
  if (dir == 0) {
    for (int yy = ly; yy < 32; yy += 8)   // S rows ti-block (bx*32+yy), cols k-block (by*32+lx)
      t[yy][lx] = S[((int64_t)lr * TILE + bx * 32 + yy) * ldd + (int64_t)k * TILE + by * 32 + lx];
    __syncthreads();
    for (int yy = ly; yy < 32; yy += 8)   // prow rows (by*32+yy), cols ti-block (bx*32+lx)
      prow[(int64_t)(by * 32 + yy) * Np + (int64_t)ti * TILE + bx * 32 + lx] = t[lx][yy];
  } else {
    for (int yy = ly; yy < 32; yy += 8)
      t[yy][lx] = prow[(int64_t)(by * 32 + yy) * Np + (int64_t)ti * TILE + bx * 32 + lx];
    __syncthreads();
    for (int yy = ly; yy < 32; yy += 8)
      S[((int64_t)lr * TILE + bx * 32 + yy) * ldd + (int64_t)k * TILE + by * 32 + lx] = t[lx][yy];
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

int g_num_sms = 0;
PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;

// 2-D int32 tensor map over rows x cols (leading dimension ld elements) with a box_rows x 128 box
ear_status_t make_map(CUtensorMap *map, const int32_t *base, int64_t rows, int64_t cols, int64_t ld, int box_rows) {
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
  cuuint64_t strides[1] = {(cuuint64_t)ld * sizeof(int32_t)};
  cuuint32_t box[2] = {(cuuint32_t)TILE, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = g_encode(map, CU_TENSOR_MAP_DATA_TYPE_INT32, 2, (void *)base, dims, strides, box, estr,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d) rows=%lld cols=%lld ld=%lld", (int)r, (long long)rows,
              (long long)cols, (long long)ld);
    return EAR_ECUDA;
  }
  return EAR_OK;
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

// Single GPU: full symmetric D (Np x Np).
ear_status_t fw_single(int32_t *D, int64_t ldd, int32_t Np, cudaStream_t st) {
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

static ear_status_t shard_xfer(const Shard &sh, int k, int32_t *prow, int dir, cudaStream_t st) {
  if (sh.nown == 0) return EAR_OK;
  dim3 g(16, sh.nt, sh.nown);
  EAR_LAUNCH(k_prow_xfer, g, 256, 0, st)(sh.S, sh.ldd, sh.d_rows, k, prow, sh.Np, dir);
  return EAR_OK;
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
ear_status_t fw_sharded_emulated(const ear_plan_s *plan, int32_t *D, int64_t ldd, int32_t Np, int32_t P,
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
  int32_t *prow = nullptr;
  if (status == EAR_OK) {
    cudaError_t e = cudaMallocAsync((void **)&prow, sizeof(int32_t) * (size_t)TILE * Np, st);
    if (e != cudaSuccess) { set_error("emulated prow: %s", cudaGetErrorString(e)); status = EAR_ENOMEM; }
  }
  CUtensorMap map_prow;
  if (status == EAR_OK) status = make_map(&map_prow, prow, TILE, Np, Np, fw_kc());
  for (int k = 0; k < nt && status == EAR_OK; ++k) {
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

}  // namespace ear
