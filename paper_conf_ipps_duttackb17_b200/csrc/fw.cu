// Phase II -- S^r = APSP(G^r) (Alg. 1 lines 4-7) as a three-phase blocked min-plus
// Floyd-Warshall (blocked FW of [23], cited at P:60) over 128 x 128 tiles on sm_100a.
//
//   D init   INF everywhere, 0 on the diagonal, atomicMin of the G^r arcs (keep the shortest of
//            parallel edges).
//   round k  phase 1  closure of the pivot tile (k,k): serial kk loop in one CTA; the matrix is
//                     symmetric (undirected G), so row kk doubles as column kk;
//            phase 2  pivot-row tiles (k,j): C = min(C, P (x) C) with the CLOSED pivot P -- a single
//                     min-plus product, no serial dependency (closure argument in DESIGN.md sec. 6);
//            phase 3  remaining tiles (i,j): C = min(C, D[i,K] (x) D[K,j]).
//   Because D is symmetric, D[i,K] = D[K,i]^T: both operands of every tile update are slices of the
//   pivot ROW block, which is also the only block a sharded round exchanges.  On one GPU only the upper
//   triangle of tiles is computed and each result is written twice (tile and transposed mirror).
//
// One persistent, dynamically scheduled, TMA-fed tile kernel (k_fw_tiles) serves phases 2 and 3 in
// two element types (fragment policies): Frag32 (int32, one VIADDMNMX per min-plus) and Frag16 (packed
// u16x2 on a copy of D capped at C16 = 0x7FFF, two min-plus per VIADDMNMX.U16x2; exact below the cap,
// DESIGN.md sec. 6d).  Both run the same lookahead schedule: round k+1's pivot chain on a per-call side
// stream while round k's remaining tiles proceed.  Every piece of per-call state (side stream, events,
// tile counters, precheck word) belongs to the call, so distinct calls on one device are independent.
#include <cooperative_groups.h>
#include <cuda.h>
#include <cudaTypedefs.h>
#include <unistd.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <vector>

#include "common.cuh"

namespace ear {
namespace {

constexpr int NT = 256;
constexpr uint32_t C16 = 0x7FFF;   // cap of the packed FW: a + b <= 0xFFFE never wraps for a, b <= C16

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

// ------------------------------------------------------------------------------ mbarrier / TMA
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

// ------------------------------------------------------------------------------ phase 1
// Closure of the int32 128x128 pivot tile at T (leading dimension ldt), in place.
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
  if (ty == 0) {   // row 0 is owned by ty = 0, r = 0
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
    const int nk = kk + 1;   // its owner publishes row nk (after this step's update) for the next step
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

// Closure of the 16-bit pivot tile (ld ldt) in place, packed like the tile kernel: thread (ty, tx) owns
// rows {ty*4 .. +3, 64 + ty*4 .. +3} as 4 row PAIRS and columns {tx*4 .. +3, 64 + tx*4 .. +3},
// c[p][q] = (T[i][j], T[i+1][j]); step kk reads row kk from shared memory -- it is also column kk, the
// tile being symmetric -- as the row-pair operand and, duplicated, as the column operand, so one
// VIADDMNMX.U16x2 relaxes two entries (values <= C16: sums <= 0xFFFE never wrap, results stay <= C16).
// About 60 registers: it fits beside the tile kernel's CTAs, which the lookahead needs.
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
    const uint2 alo = *reinterpret_cast<const uint2 *>(rb + ty * 4);
    const uint2 ahi = *reinterpret_cast<const uint2 *>(rb + 64 + ty * 4);
    const uint2 blo = *reinterpret_cast<const uint2 *>(rb + tx * 4);
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
    const int nk = kk + 1;
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

// ------------------------------------------------------------------------------ phases 2 and 3
// Tile sets of one launch (round k):
//   MODE_PIVOT_ROW   tiles (k, j != k)                        -- phase 2, single GPU
//   MODE_UPPER       upper tiles outside row/column k         -- phase 3, single GPU
//   MODE_CROSS       upper tiles of row/column k+1 (not k)    -- lookahead: first part of phase 3
//   MODE_REST        upper tiles outside rows/columns k, k+1  -- lookahead: the rest
//   MODE_LIST        a rank's owned upper tiles outside row/column k (C addressed by local tile row)
//   MODE_LIST_CROSS / MODE_LIST_REST   the same split of MODE_LIST
//   MODE_PIECES      phase 2 on the pivot-row pieces a rank contributes: tiles (k, orow[i]) for its mk
//                    owned rows above k, then (k, k+1 ..) when it owns row k (posk >= 0)
enum { MODE_PIVOT_ROW = 0, MODE_UPPER = 1, MODE_LIST = 2, MODE_CROSS = 3, MODE_REST = 4, MODE_LIST_CROSS = 5,
       MODE_LIST_REST = 6, MODE_PIECES = 7 };

struct TileJob {
  void *C;           // matrix holding the C tiles (local tile rows), leading dimension ldc (elements)
  int64_t ldc;
  int32_t a_row0;    // row of the pivot row block inside the A operand's tensor map
  int32_t b_row0;    // ... inside the B operand's map
  int32_t k;         // pivot tile index
  int32_t nt;        // tiles per dimension (Np / 128)
  int32_t ti0;       // first tile row held by C (lr = ti - ti0 outside the list modes)
  int32_t mode;
  int32_t mirror;    // also write the transposed result into tile (tj, ti) (single GPU)
  int64_t ntiles;    // tiles in this launch
  // list modes: the rank's owned tile rows (ascending), the static prefix sums of their upper-tile
  // counts (nt - ti), and per round: mk = #owned rows < k, posk / posk1 = position of row k / k+1 in
  // the owned list or -1
  const int32_t *orow;
  const int64_t *opre;
  int32_t nown, mk, posk, posk1;
  int32_t *counter;  // {next tile, CTAs done}: zero at launch, reset by the launch's last CTA
};

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

// Fragment policies of the tile kernel: C tile in registers, operand chunks (KC rows of the pivot row
// block, A^T for the tile's rows, B for its columns) from shared memory.
//
// Frag32: 256 threads, 8 x 8 int32 per thread (rows {ty*4 .. +3, 64 + ty*4 .. +3}, columns
// {tx*4 .. +3, 64 + tx*4 .. +3}), 64-deep chunks, 2-stage ring (128 KB), one CTA per SM: chosen by
// measurement on the B200 (round 1, profiles/r01_fw_variants.txt: 88 % of the int32 VIADDMNMX peak).
struct Frag32 {
  using E = int32_t;
  static constexpr int NTH = 256, KC = 64, STAGES = 2, MINB = 1;
  static constexpr int A_BYTES = KC * TILE * 4, B_BYTES = KC * TILE * 4;
  struct Acc {
    int32_t c[8][8];
  };
  __device__ static int row(int r, int ty) { return (r < 4 ? 0 : 64) + ty * 4 + (r & 3); }
  __device__ static void load(Acc &a, const E *Ct, int64_t ldc, int tid) {
    const int tx = tid & 15, ty = tid >> 4;
#pragma unroll
    for (int r = 0; r < 8; ++r) {
      const int i = row(r, ty);
      const int4 lo = *reinterpret_cast<const int4 *>(Ct + (int64_t)i * ldc + tx * 4);
      const int4 hi = *reinterpret_cast<const int4 *>(Ct + (int64_t)i * ldc + 64 + tx * 4);
      a.c[r][0] = lo.x; a.c[r][1] = lo.y; a.c[r][2] = lo.z; a.c[r][3] = lo.w;
      a.c[r][4] = hi.x; a.c[r][5] = hi.y; a.c[r][6] = hi.z; a.c[r][7] = hi.w;
    }
  }
  __device__ static void chunk(Acc &a, const uint8_t *sa, const uint8_t *sb, int tid) {
    const int tx = tid & 15, ty = tid >> 4;
    const int32_t *a_s = reinterpret_cast<const int32_t *>(sa), *b_s = reinterpret_cast<const int32_t *>(sb);
#pragma unroll 16
    for (int kk = 0; kk < KC; ++kk) {
      const int4 alo = *reinterpret_cast<const int4 *>(a_s + kk * TILE + ty * 4);
      const int4 ahi = *reinterpret_cast<const int4 *>(a_s + kk * TILE + 64 + ty * 4);
      const int4 blo = *reinterpret_cast<const int4 *>(b_s + kk * TILE + tx * 4);
      const int4 bhi = *reinterpret_cast<const int4 *>(b_s + kk * TILE + 64 + tx * 4);
      const int32_t av[8] = {alo.x, alo.y, alo.z, alo.w, ahi.x, ahi.y, ahi.z, ahi.w};
      const int32_t bv[8] = {blo.x, blo.y, blo.z, blo.w, bhi.x, bhi.y, bhi.z, bhi.w};
#pragma unroll
      for (int r = 0; r < 8; ++r)
#pragma unroll
        for (int q = 0; q < 8; ++q) a.c[r][q] = mp(av[r], bv[q], a.c[r][q]);
    }
  }
  __device__ static void store(const Acc &a, E *Ct, int64_t ldc, int tid) {
    const int tx = tid & 15, ty = tid >> 4;
#pragma unroll
    for (int r = 0; r < 8; ++r) {
      const int i = row(r, ty);
      *reinterpret_cast<int4 *>(Ct + (int64_t)i * ldc + tx * 4) = make_int4(a.c[r][0], a.c[r][1], a.c[r][2], a.c[r][3]);
      *reinterpret_cast<int4 *>(Ct + (int64_t)i * ldc + 64 + tx * 4) = make_int4(a.c[r][4], a.c[r][5], a.c[r][6], a.c[r][7]);
    }
  }
  __device__ static void store_mirror(const Acc &a, E *Mt, int64_t ldc, int tid) {
    const int tx = tid & 15, ty = tid >> 4;
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const int j = (q < 4 ? 0 : 64) + tx * 4 + (q & 3);
      *reinterpret_cast<int4 *>(Mt + (int64_t)j * ldc + ty * 4) = make_int4(a.c[0][q], a.c[1][q], a.c[2][q], a.c[3][q]);
      *reinterpret_cast<int4 *>(Mt + (int64_t)j * ldc + 64 + ty * 4) = make_int4(a.c[4][q], a.c[5][q], a.c[6][q], a.c[7][q]);
    }
  }
};

// Frag16: 128 threads, 16 rows x 8 columns each as 8 row PAIRS x 8 columns, c[p][q] = (C[i][j], C[i+1][j])
// packed; A chunks are u16 rows of the pivot row block (row pairs are adjacent u16: one register), B
// chunks rows of its copy with every value duplicated into both halves, so one VIADDMNMX.U16x2 updates
// two entries with no unpacking in the inner loop.  32-deep chunks, 2-stage ring (48 KB), 3 CTAs per
// SM: chosen by a 17-variant sweep on the B200 (round 1, profiles/r01_fw16_variants.jsonl).
struct Frag16 {
  using E = uint16_t;
  static constexpr int NTH = 128, KC = 32, STAGES = 2, MINB = 3;
  static constexpr int A_BYTES = KC * TILE * 2, B_BYTES = KC * TILE * 4;
  struct Acc {
    uint32_t c[8][8];
  };
  __device__ static int row(int r2, int ty) { return (r2 < 4 ? 0 : 64) + ty * 8 + (r2 & 3) * 2; }
  __device__ static void load(Acc &a, const E *Ct, int64_t ldc, int tid) {
    const int tx = tid & 15, ty = tid >> 4;
#pragma unroll
    for (int r2 = 0; r2 < 8; ++r2) {
      const int i = row(r2, ty);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const uint2 v = *reinterpret_cast<const uint2 *>(Ct + (int64_t)i * ldc + h * 64 + tx * 4);
        const uint2 w = *reinterpret_cast<const uint2 *>(Ct + (int64_t)(i + 1) * ldc + h * 64 + tx * 4);
        a.c[r2][h * 4 + 0] = __byte_perm(v.x, w.x, 0x5410);
        a.c[r2][h * 4 + 1] = __byte_perm(v.x, w.x, 0x7632);
        a.c[r2][h * 4 + 2] = __byte_perm(v.y, w.y, 0x5410);
        a.c[r2][h * 4 + 3] = __byte_perm(v.y, w.y, 0x7632);
      }
    }
  }
  __device__ static void chunk(Acc &a, const uint8_t *sa, const uint8_t *sb, int tid) {
    const int tx = tid & 15, ty = tid >> 4;
    const uint16_t *a_s = reinterpret_cast<const uint16_t *>(sa);
    const uint32_t *b_s = reinterpret_cast<const uint32_t *>(sb);
#pragma unroll 16
    for (int kk = 0; kk < KC; ++kk) {
      const uint4 alo = *reinterpret_cast<const uint4 *>(a_s + kk * TILE + ty * 8);
      const uint4 ahi = *reinterpret_cast<const uint4 *>(a_s + kk * TILE + 64 + ty * 8);
      const uint32_t av[8] = {alo.x, alo.y, alo.z, alo.w, ahi.x, ahi.y, ahi.z, ahi.w};
      const uint4 blo = *reinterpret_cast<const uint4 *>(b_s + kk * TILE + tx * 4);
      const uint4 bhi = *reinterpret_cast<const uint4 *>(b_s + kk * TILE + 64 + tx * 4);
      const uint32_t bv[8] = {blo.x, blo.y, blo.z, blo.w, bhi.x, bhi.y, bhi.z, bhi.w};
#pragma unroll
      for (int r2 = 0; r2 < 8; ++r2)
#pragma unroll
        for (int q = 0; q < 8; ++q) a.c[r2][q] = __viaddmin_u16x2(av[r2], bv[q], a.c[r2][q]);
    }
  }
  __device__ static void store(const Acc &a, E *Ct, int64_t ldc, int tid) {
    const int tx = tid & 15, ty = tid >> 4;
#pragma unroll
    for (int r2 = 0; r2 < 8; ++r2) {
      const int i = row(r2, ty);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const uint32_t *cc = &a.c[r2][h * 4];
        *reinterpret_cast<uint2 *>(Ct + (int64_t)i * ldc + h * 64 + tx * 4) =
            make_uint2(__byte_perm(cc[0], cc[1], 0x5410), __byte_perm(cc[2], cc[3], 0x5410));
        *reinterpret_cast<uint2 *>(Ct + (int64_t)(i + 1) * ldc + h * 64 + tx * 4) =
            make_uint2(__byte_perm(cc[0], cc[1], 0x7632), __byte_perm(cc[2], cc[3], 0x7632));
      }
    }
  }
  __device__ static void store_mirror(const Acc &a, E *Mt, int64_t ldc, int tid) {
    const int tx = tid & 15, ty = tid >> 4;
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const int j = (q < 4 ? 0 : 64) + tx * 4 + (q & 3);
#pragma unroll
      for (int h = 0; h < 2; ++h)
        *reinterpret_cast<uint4 *>(Mt + (int64_t)j * ldc + h * 64 + ty * 8) =
            make_uint4(a.c[h * 4][q], a.c[h * 4 + 1][q], a.c[h * 4 + 2][q], a.c[h * 4 + 3][q]);
    }
  }
};

// The tile kernel.  Persistent CTAs, dynamically scheduled: a CTA takes its next tile from a global
// counter when it issues that tile's first TMA chunk (round 1 measured the static assignment ending
// its CTAs between 43 % and 100 % of a launch -- the CTAs of an SM run at different speeds), and
// publishes it, tagged with its sequence number q, in tslot[q & 1]; the ring depth (2) never exceeds
// the chunks per tile, so a slot is rewritten only after every warp has read it.  Operand chunks
// stream through a STAGES-deep shared-memory ring filled by cp.async.bulk.tensor (TMA), completion
// tracked by mbarriers; a stage is refilled by the LAST warp to finish reading it (a shared counter),
// so no CTA-wide barrier sits in the main loop.  The last CTA to finish resets the counter pair.
template <class F>
__global__ void __launch_bounds__(F::NTH, F::MINB)
    k_fw_tiles(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, const TileJob J) {
  constexpr int KC = F::KC, NCHUNK = TILE / KC, STAGES = F::STAGES, NW = F::NTH / 32;
  static_assert(NCHUNK >= STAGES, "tile slots are rewritten only after every warp has read them");
  constexpr int32_t NONE = 0xFFFFF;
  using E = typename F::E;
  extern __shared__ __align__(128) uint8_t smem[];
  uint8_t *sA = smem;
  uint8_t *sB = sA + STAGES * F::A_BYTES;
  uint64_t *full = reinterpret_cast<uint64_t *>(sB + STAGES * F::B_BYTES);
  int32_t *cnt = reinterpret_cast<int32_t *>(full + STAGES);   // [STAGES] warps done with the stage
  int32_t *tslot = cnt + STAGES;                               // [2] (q << 20) | tile
  const int tid = threadIdx.x, lane = tid & 31;
  auto issue = [&](int c, int st) {   // chunk c of this CTA's sequence into stage st (one thread)
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
    decode_tile(J, t, pti, ptj, plr);
    mbar_arrive_tx(&full[st], F::A_BYTES + F::B_BYTES);
    tma_load_2d(sA + st * F::A_BYTES, &tmA, pti * TILE, J.a_row0 + kc * KC, &full[st]);
    tma_load_2d(sB + st * F::B_BYTES, &tmB, ptj * TILE, J.b_row0 + kc * KC, &full[st]);
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

  int g = 0;
  for (int q = 0;; ++q) {
    mbar_wait(&full[g % STAGES], (uint32_t)((g / STAGES) & 1));
    const int32_t v = tslot[q & 1] & NONE;
    if (v == NONE) break;
    int ti, tj, lr;
    decode_tile(J, v, ti, tj, lr);
    E *Ct = static_cast<E *>(J.C) + (int64_t)lr * TILE * J.ldc + (int64_t)tj * TILE;
    typename F::Acc acc;
    F::load(acc, Ct, J.ldc, tid);   // C straight into registers (its latency overlaps the in-flight TMA)
#pragma unroll 1
    for (int kc = 0; kc < NCHUNK; ++kc, ++g) {
      const int st = g % STAGES;
      if (kc > 0) mbar_wait(&full[st], (uint32_t)((g / STAGES) & 1));
      F::chunk(acc, sA + st * F::A_BYTES, sB + st * F::B_BYTES, tid);
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
    F::store(acc, Ct, J.ldc, tid);
    if (J.mirror && ti != tj)
      F::store_mirror(acc, static_cast<E *>(J.C) + (int64_t)tj * TILE * J.ldc + (int64_t)ti * TILE, J.ldc, tid);
  }
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    if (atomicAdd(J.counter + 1, 1) == (int)gridDim.x - 1) {   // the last CTA resets the pair
      J.counter[0] = 0;
      J.counter[1] = 0;
      __threadfence();
    }
  }
}

// ------------------------------------------------------------------------------ 16-bit conversions
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

// capped entries of connected pairs (lab[i] == lab[j]; only vertices < n_real; labels may be null:
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

// largest finite entry of a distance row (the cap precheck)
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

// Pd[r][c] = P16[r][c] duplicated into both halves (the B operand of the packed product); 128 x Np
__global__ void k_dup16(const uint16_t *__restrict__ P16, int32_t Np, uint32_t *__restrict__ Pd) {
  const int64_t total = (int64_t)TILE * (Np / 4);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const uint2 v = reinterpret_cast<const uint2 *>(P16)[i];
    reinterpret_cast<uint4 *>(Pd)[i] = make_uint4((v.x & 0xFFFFu) * 0x10001u, (v.x >> 16) * 0x10001u,
                                                  (v.y & 0xFFFFu) * 0x10001u, (v.y >> 16) * 0x10001u);
  }
}

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

// k_check16 over a rank's owned UPPER tiles (the authoritative ones; D is symmetric, so the ranks
// together cover every pair): a capped entry of a connected pair sets *flag = -1
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

// ------------------------------------------------------------------------------ sharding kernels
// Pivot-row block <-> a rank's owned storage, round k (L: 128 x Np, leading dimension Np).
//   dir = 0 (gather):  L[:, ti-block] = S(ti, k)^T for owned ti < k; L[:, j >= k] = S(k, j) if row k owned
//   dir = 1 (scatter): the inverse, from the completed (phase-2-updated) block
// Grid (16 sub-blocks of 32 x 32, npieces), 256 threads: pieces [0, nrow) are the tiles j = k + y of the
// pivot row when this rank owns it (nrow = nt - k, local row posk), the next mk the owned rows ti < k.
template <class E>
__global__ void k_prow_xfer(E *S, int64_t ldd, const int32_t *orow, int32_t k, int32_t nt, int32_t posk, E *L,
                            int32_t Np, int dir) {
  __shared__ E t[32][33];
  const int nrow = posk >= 0 ? nt - k : 0;
  const int y = blockIdx.y;
  const int bx = blockIdx.x & 3, by = blockIdx.x >> 2;         // 32 x 32 sub-block (bx: x, by: y)
  const int lx = threadIdx.x & 31, ly = threadIdx.x >> 5;      // 32 x 8 threads
  if (y < nrow) {              // the pivot row's upper part: plain copy, tiles j >= k
    const int lr = posk, tj = k + y;
    for (int yy = ly; yy < 32; yy += 8) {
      const int64_t row = by * 32 + yy, col = (int64_t)tj * TILE + bx * 32 + lx;
      E *sp = S + ((int64_t)lr * TILE + row) * ldd + col;
      E *pp = L + row * Np + col;
      if (dir == 0) *pp = *sp; else *sp = *pp;
    }
    return;
  }
  const int lr = y - nrow, ti = orow[lr];   // owned row below the pivot: tile (ti, k) <-> L[:, ti-block]^T
  if (dir == 0) {
    for (int yy = ly; yy < 32; yy += 8)   // S rows ti-block (bx*32+yy), cols k-block (by*32+lx)
      t[yy][lx] = S[((int64_t)lr * TILE + bx * 32 + yy) * ldd + (int64_t)k * TILE + by * 32 + lx];
    __syncthreads();
    for (int yy = ly; yy < 32; yy += 8)   // L rows (by*32+yy), cols ti-block (bx*32+lx)
      L[(int64_t)(by * 32 + yy) * Np + (int64_t)ti * TILE + bx * 32 + lx] = t[lx][yy];
  } else {
    for (int yy = ly; yy < 32; yy += 8)
      t[yy][lx] = L[(int64_t)(by * 32 + yy) * Np + (int64_t)ti * TILE + bx * 32 + lx];
    __syncthreads();
    for (int yy = ly; yy < 32; yy += 8)
      S[((int64_t)lr * TILE + bx * 32 + yy) * ldd + (int64_t)k * TILE + by * 32 + lx] = t[lx][yy];
  }
}

// The per-round broadcast of the pieces: this rank's column blocks of the phase-2-updated pivot row
// block (k .. nt-1 when it owns row k, then its owned rows below k -- see k_prow_xfer) are copied from
// L into the same positions of every destination block dst.p[d] (the peers' stage buffers, mapped over
// NVLink, and its own).  Grid (max(npieces, 1), 4 row quarters).  With `counter` the last CTA to finish
// raises flag slot `slot` of every window in `flags` to `value` (system-scope release after every CTA's
// stores are fenced: a peer that sees the flag sees the data).
template <class E>
__global__ void k_push_pieces(const E *__restrict__ L, int32_t Np, int32_t k, int32_t nt, int32_t posk, int32_t mk,
                              const int32_t *__restrict__ orow, PeerPtrs dst, int32_t *counter, PeerPtrs flags,
                              int32_t slot, uint64_t value) {
  const int nrow = posk >= 0 ? nt - k : 0;
  const int y = blockIdx.x;
  if (y < nrow + mk) {
    const int cb = y < nrow ? k + y : orow[y - nrow];
    constexpr int V = 16 / (int)sizeof(E);   // elements per 16-byte vector
    constexpr int PER_ROW = TILE / V;
    for (int i = threadIdx.x; i < 32 * PER_ROW; i += blockDim.x) {
      const int r = blockIdx.y * 32 + i / PER_ROW, c = (i % PER_ROW) * V;
      const int64_t off = (int64_t)r * Np + (int64_t)cb * TILE + c;
      const uint4 v = *reinterpret_cast<const uint4 *>(L + off);
      for (int d = 0; d < dst.n; ++d) *reinterpret_cast<uint4 *>(reinterpret_cast<E *>(dst.p[d]) + off) = v;
    }
  }
  if (!counter) return;
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0 && atomicAdd(counter, 1) == (int)(gridDim.x * gridDim.y) - 1) {
    *counter = 0;   // the next push on this stream starts from zero
    __threadfence_system();
    for (int d = 0; d < flags.n; ++d) {
      uint64_t *f = reinterpret_cast<uint64_t *>(flags.p[d]) + slot;
      asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(value) : "memory");
    }
  }
}

// the range-check bit of this rank -> CHECK slot `slot` of every window, value (seq << 1) | bad
__global__ void k_check_push(const int32_t *flag, PeerPtrs wins, int32_t slot, uint64_t seq) {
  const uint64_t v = (seq << 1) | (uint64_t)(*flag < 0 ? 1 : 0);
  __threadfence_system();
  for (int d = threadIdx.x; d < wins.n; d += blockDim.x) {
    uint64_t *f = reinterpret_cast<uint64_t *>(wins.p[d]) + slot;
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(v) : "memory");
  }
}
// OR of the ranks' bits (this rank's window, slots [slot, slot + P)) -> *flag = -1 if any is set
__global__ void k_check_fold(const uint64_t *slots, int32_t P, int32_t *flag) {
  if (threadIdx.x == 0) {
    int any = 0;
    for (int p = 0; p < P; ++p) {
      uint64_t v;
      asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(slots + p) : "memory");
      any |= (int)(v & 1);
    }
    *flag = any ? -1 : 0;
  }
}

// owned upper tiles (ti, tj >= ti) -> full D, and their transposed mirrors (tj, ti)  (emulated ranks)
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

// The all-gather of D: every tile (ti, tj) of the full matrix Df is read from the window region of the
// rank that owns it -- tile row ti when tj >= ti (owner of row ti under the zig-zag, local row position
// = 2 * (ti / 2P) + (ti mod 2P >= P)), else the transpose of upper tile (tj, ti).  Regions hold the
// owned tile rows with leading dimension Np.  Grid (nt, nt), 256 threads, 32 x 32 sub-blocks.
__global__ void k_gather_pull(PeerPtrs regions, int32_t P, int32_t Np, int32_t *__restrict__ Df, int64_t ldf) {
  __shared__ int32_t t[32][33];
  const int ti = blockIdx.y, tj = blockIdx.x;
  const int up = tj >= ti;
  const int sr = up ? ti : tj, sc = up ? tj : ti;   // the authoritative tile (sr, sc), sc >= sr
  const int o = sr % (2 * P);
  const int rank = o < P ? o : 2 * P - 1 - o, pos = 2 * (sr / (2 * P)) + (o >= P ? 1 : 0);
  const int32_t *src = reinterpret_cast<const int32_t *>(regions.p[rank]) + (int64_t)pos * TILE * Np + (int64_t)sc * TILE;
  int32_t *dst = Df + (int64_t)ti * TILE * ldf + (int64_t)tj * TILE;
  const int lx = threadIdx.x & 31, ly = threadIdx.x >> 5;
  if (up) {
    for (int i = threadIdx.x; i < TILE * TILE / 4; i += blockDim.x) {
      const int r = i >> 5, c = (i & 31) * 4;
      *reinterpret_cast<int4 *>(dst + (int64_t)r * ldf + c) = *reinterpret_cast<const int4 *>(src + (int64_t)r * Np + c);
    }
    return;
  }
  for (int sb = 0; sb < 16; ++sb) {   // dst (r, c) = src (c, r)
    const int bx = sb & 3, by = sb >> 2;
    __syncthreads();
    for (int yy = ly; yy < 32; yy += 8) t[yy][lx] = src[(int64_t)(bx * 32 + yy) * Np + by * 32 + lx];
    __syncthreads();
    for (int yy = ly; yy < 32; yy += 8) dst[(int64_t)(by * 32 + yy) * ldf + bx * 32 + lx] = t[lx][yy];
  }
}

// connected-component labels (min vertex id) of the reduced graph by hooking + pointer jumping
// connected components of G^r in one cooperative launch: hooking of roots (smaller id wins) and pointer
// jumping, separated by grid barriers, until a hooking pass changes nothing; labels = smallest vertex id
// of the component.  st[0..2]: rotating per-pass change flags
__global__ void k_cc_coop(const int32_t *__restrict__ u, const int32_t *__restrict__ v, int64_t E, int32_t *lab,
                          int32_t n, int32_t *st) {
  namespace cg = cooperative_groups;
  cg::grid_group grid = cg::this_grid();
  const int64_t tid0 = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t x = tid0; x < n; x += stride) lab[x] = (int32_t)x;
  if (tid0 == 0) st[0] = st[1] = st[2] = 0;
  grid.sync();
  for (int it = 0; it < 4 * 64; ++it) {
    const int f = it % 3;
    int ch = 0;
    for (int64_t i = tid0; i < E; i += stride) {
      const int32_t a = lab[u[i]], b = lab[v[i]];
      if (a != b) {
        const int32_t hi = max(a, b), lo = min(a, b);
        if (atomicMin(&lab[hi], lo) > lo) ch = 1;
      }
    }
    if (__syncthreads_or(ch) && threadIdx.x == 0) st[f] = 1;
    if (tid0 == 0) st[(it + 1) % 3] = 0;   // read two passes ago, before the last barrier
    grid.sync();
    for (int64_t x = tid0; x < n; x += stride) {
      int32_t l = lab[x];
      while (lab[l] != l) l = lab[l];
      lab[x] = l;
    }
    grid.sync();
    if (!st[f]) return;
  }
}


// EAR_DEBUG_RACE_US (test knob, tests/test_concurrency_gpu.py): a device-side spin of that length ahead
// of each cross-tile launch keeps the device behind the host, and a host sleep of the same length
// between recording the cross-tile event and the side stream's wait on it widens the window in which
// another FW call on the device could interleave.  Per-call lookahead state makes the result immune.
__global__ void k_debug_spin(long long ns) {
  const long long t0 = clock64();
  while (clock64() - t0 < ns * 2) {
  }
}
int debug_race_us() {
  const char *e = getenv("EAR_DEBUG_RACE_US");
  return e ? atoi(e) : 0;
}
void debug_gpu_delay(cudaStream_t st) {
  if (debug_race_us() > 0) k_debug_spin<<<1, 32, 0, st>>>((long long)debug_race_us() * 1000);
}
void debug_host_delay() {
  if (debug_race_us() > 0) usleep((useconds_t)debug_race_us());
}

// ============================================================================== host side
int grid_for(int64_t n) { return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 16)); }

int env_int(const char *name, int dflt) {
  const char *e = getenv(name);
  return e ? atoi(e) : dflt;
}

PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;
std::once_flag g_encode_once;

// 2-D tensor map over rows x cols (leading dimension ld elements of elem bytes) with a box_rows x 128 box
ear_status_t make_map(CUtensorMap *map, int elem, const void *base, int64_t rows, int64_t cols, int64_t ld,
                      int box_rows) {
  std::call_once(g_encode_once, [] {
    cudaDriverEntryPointQueryResult q;
    void *fn = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      g_encode = (PFN_cuTensorMapEncodeTiled_v12000)fn;
    cudaGetLastError();
  });
  if (!g_encode) {
    set_error("cuTensorMapEncodeTiled unavailable");
    return EAR_ECUDA;
  }
  const CUtensorMapDataType dt = elem == 2 ? CU_TENSOR_MAP_DATA_TYPE_UINT16
                                           : CU_TENSOR_MAP_DATA_TYPE_INT32;   // u32 operands: same bits
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

template <class F>
constexpr int smem_bytes() {
  return F::STAGES * (F::A_BYTES + F::B_BYTES) + F::STAGES * 8 + F::STAGES * 4 + 8;
}

// resident CTAs per SM of the tile kernel (per device, cached)
template <class F>
int tiles_per_sm() {
  static int cache[64] = {};
  static std::mutex mu;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(mu);
  if (dev >= 0 && dev < 64 && cache[dev]) return cache[dev];
  int per = 0;
  if (smem_attr((const void *)k_fw_tiles<F>, smem_bytes<F>()) != cudaSuccess ||
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_fw_tiles<F>, F::NTH, smem_bytes<F>()) != cudaSuccess)
    per = 0;
  cudaGetLastError();
  per = std::max(per, 1);
  if (dev >= 0 && dev < 64) cache[dev] = per;
  return per;
}

template <class F>
ear_status_t launch_tiles(const CUtensorMap &mA, const CUtensorMap &mB, TileJob J, int64_t ntiles, int32_t *counter,
                          cudaStream_t st, int reserve = 0) {
  if (ntiles <= 0) return EAR_OK;
  if (ntiles >= 0xFFFFF) {
    set_error("fw: %lld tiles in one launch exceed the tile kernel's 20-bit tile index", (long long)ntiles);
    return EAR_EUNSUPPORTED;
  }
  EAR_CUDA_TRY(smem_attr((const void *)k_fw_tiles<F>, smem_bytes<F>()));
  J.ntiles = ntiles;
  J.counter = counter;
  const int64_t slots = (int64_t)num_sms() * tiles_per_sm<F>();
  const int64_t grid = std::min<int64_t>(ntiles, std::max<int64_t>(1, slots - reserve));
  EAR_LAUNCH(k_fw_tiles<F>, (unsigned)grid, F::NTH, smem_bytes<F>(), st)(mA, mB, J);
  return EAR_OK;
}

// CTA slots the rest-of-round launch leaves to the next round's pivot chain.  The persistent,
// dynamically scheduled tile kernel frees no slot before it drains, so the chain's phase-2 tiles (p2)
// run on the reserved slots alongside the rest (rest tiles): enough slots that they finish no later,
// p2 / R <= rest / (slots - R).  EAR_FW_RESERVE overrides (round 1 measured 4 best on cfg4's packed FW,
// which is what the rule gives there, profiles/r01y_fw16_dyn.jsonl).
template <class F>
int lookahead_reserve(int64_t rest, int64_t p2) {
  const int forced = env_int("EAR_FW_RESERVE", -1);
  if (forced >= 0) return forced;
  const int64_t slots = (int64_t)num_sms() * tiles_per_sm<F>();
  const int64_t r = (slots * p2 + rest + p2 - 1) / std::max<int64_t>(rest + p2, 1);
  return (int)std::min<int64_t>(std::max<int64_t>(r, 1), slots / 2);
}

// ---- per-call lookahead state: side stream, events and the precheck's mapped word, from a pool per
// device (a context is held by one FW call from start to end: nothing is shared between calls)
struct FwCtx {
  int dev = -1;
  cudaStream_t side = nullptr;
  cudaEvent_t ev_cross = nullptr, ev_pivot = nullptr;
  int32_t *h_word = nullptr;   // mapped pinned
};
std::mutex g_ctx_mu;
std::vector<FwCtx *> g_ctx_free;

ear_status_t ctx_acquire(FwCtx **out) {
  int dev = 0;
  EAR_CUDA_TRY(cudaGetDevice(&dev));
  {
    std::lock_guard<std::mutex> lk(g_ctx_mu);
    for (size_t i = 0; i < g_ctx_free.size(); ++i)
      if (g_ctx_free[i]->dev == dev) {
        *out = g_ctx_free[i];
        g_ctx_free.erase(g_ctx_free.begin() + (long)i);
        return EAR_OK;
      }
  }
  FwCtx *c = new FwCtx;
  c->dev = dev;
  int lo = 0, hi = 0;   // the pivot chain gets the highest priority: its CTAs take the first free slots
  cudaError_t e = cudaDeviceGetStreamPriorityRange(&lo, &hi);
  if (e == cudaSuccess) e = cudaStreamCreateWithPriority(&c->side, cudaStreamNonBlocking, hi);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_cross, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_pivot, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaHostAlloc((void **)&c->h_word, sizeof(int32_t), cudaHostAllocMapped | cudaHostAllocPortable);
  if (e != cudaSuccess) {
    set_error("fw: lookahead context: %s", cudaGetErrorString(e));
    delete c;
    return EAR_ECUDA;
  }
  *out = c;
  return EAR_OK;
}
void ctx_release(FwCtx *c) {
  if (!c) return;
  std::lock_guard<std::mutex> lk(g_ctx_mu);
  g_ctx_free.push_back(c);
}
struct CtxLease {
  FwCtx *c = nullptr;
  ~CtxLease() { ctx_release(c); }
};

// Cap precheck of the packed FW: one single-source SSSP row of reduced vertex 0 on a helper stream,
// its eccentricity (a lower bound on the largest finite distance) read back asynchronously into the
// call's mapped word.  start() does nothing without a plan, for a small FW (< 64 tiles) or with
// EAR_FW16_PRECHECK=0; hopeless() waits for the row and says whether it reached the cap.  The row is
// exact and deterministic, so every rank of a sharded FW takes the same decision without a collective.
struct Precheck {
  cudaStream_t hs = nullptr;
  cudaEvent_t ev = nullptr;
  int32_t *row = nullptr;
  int32_t *h = nullptr;
  bool on = false;
  void start(ear_plan_s *plan, int32_t Np, int32_t n_real, int nt, int32_t *h_word) {
    h = h_word;
    if (!plan || nt < 64 || env_int("EAR_FW16_PRECHECK", 1) == 0 || !h) return;
    on = cudaStreamCreateWithFlags(&hs, cudaStreamNonBlocking) == cudaSuccess &&
         cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) == cudaSuccess &&
         cudaMallocAsync((void **)&row, sizeof(int32_t) * ((size_t)Np + 1), hs) == cudaSuccess &&
         dev_memset(row + Np, 0, sizeof(int32_t), hs) == cudaSuccess &&
         sssp_rows(plan, row, Np, Np, 0, 1, nullptr, hs) == EAR_OK;
    if (on) {
      EAR_LAUNCH(k_row_far, grid_for(n_real), 256, 0, hs)(row, n_real, row + Np);
      on = readback_direct(h, row + Np, sizeof(int32_t), hs) == cudaSuccess && cudaEventRecord(ev, hs) == cudaSuccess;
    }
    if (!on) cudaGetLastError();
  }
  bool hopeless() { return on && cudaEventSynchronize(ev) == cudaSuccess && *h >= (int32_t)C16; }
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

// stream-ordered scratch of one FW call, freed in stream order at scope exit
struct Scratch {
  cudaStream_t st;
  std::vector<void *> ptrs;
  explicit Scratch(cudaStream_t s) : st(s) {}
  template <class T>
  bool get(T **p, size_t elems) {
    *p = nullptr;
    if (cudaMallocAsync((void **)p, sizeof(T) * std::max<size_t>(elems, 1), st) != cudaSuccess) {
      cudaGetLastError();
      *p = nullptr;
      return false;
    }
    ptrs.push_back(*p);
    return true;
  }
  ~Scratch() {
    for (void *p : ptrs) cudaFreeAsync(p, st);
  }
};

// ============================================================================== single GPU
// Single-GPU lookahead schedule for element policy F on the full symmetric matrix (int32: D itself;
// packed: the capped u16 copy D16 with its duplicated pivot-row buffers Pd[2]).  Round k's phase 3 is
// split into the tiles of row/column k+1 (MODE_CROSS, first) and the rest (MODE_REST); once the cross
// tiles are done, round k+1's pivot chain -- phase 1 on tile (k+1, k+1), phase 2 on row k+1 (packed:
// with its duplicated copies) -- runs on the call's side stream while the rest of round k proceeds
// (leaving it a few CTA slots); round k+1's phase 3 waits for the chain.  The two streams touch disjoint
// tiles (the rest skips rows/columns k, k+1; phase 2's mirrors land in column k+1).  With a precheck
// (packed only) the schedule stops after round 3 when the cap is certainly reached (*hopeless).
template <class F>
ear_status_t fw_single_sched(typename F::E *D, int64_t ldd, int32_t Np, uint32_t *Pd, FwCtx *ctx, int32_t *cnt,
                             cudaStream_t st, Precheck *pc, bool *hopeless) {
  constexpr bool PACKED = sizeof(typename F::E) == 2;
  using E = typename F::E;
  const int nt = Np / TILE;
  const double tile_ops = (double)TILE * TILE * TILE;
  const bool lookahead = env_int("EAR_FW_LOOKAHEAD", 1) != 0;
  *hopeless = false;
  CUtensorMap mA, mB[2];
  EAR_TRY(make_map(&mA, (int)sizeof(E), D, Np, Np, ldd, F::KC));
  if (PACKED)
    for (int b = 0; b < 2; ++b) EAR_TRY(make_map(&mB[b], 4, Pd + (size_t)b * TILE * Np, TILE, Np, Np, F::KC));
  const int64_t ndup = (int64_t)TILE * (Np / 4);
  int32_t *cnt_main = cnt, *cnt_side = cnt + 2;
  // phases 1 and 2 of round k on stream q
  auto pivot = [&](int k, cudaStream_t q) -> ear_status_t {
    E *Pk = D + (int64_t)k * TILE * ldd;   // pivot row block
    const bool on_side = q != st;          // lookahead: overlapped with phase 3, reported apart
    int s1 = prof_begin(on_side ? PK_FW_SIDE_P1 : PK_FW_P1, q);
    if (PACKED)
      EAR_LAUNCH(k_fw_phase1_16, 1, NT, 0, q)(reinterpret_cast<uint16_t *>(Pk) + (int64_t)k * TILE, ldd);
    else
      EAR_LAUNCH(k_fw_phase1, 1, NT, 0, q)(reinterpret_cast<int32_t *>(Pk) + (int64_t)k * TILE, ldd);
    prof_end(s1, q, tile_ops);
    int s2 = prof_begin(on_side ? PK_FW_SIDE_P2 : PK_FW_P2, q);
    uint32_t *Pdk = Pd ? Pd + (size_t)(k & 1) * TILE * Np : nullptr;
    if (PACKED)   // B of phase 2: the pre-phase-2 row, duplicated
      EAR_LAUNCH(k_dup16, grid_for(ndup), 256, 0, q)(reinterpret_cast<const uint16_t *>(Pk), Np, Pdk);
    TileJob J{D, ldd, k * TILE, PACKED ? 0 : k * TILE, k, nt, 0, MODE_PIVOT_ROW, 1};
    EAR_TRY(launch_tiles<F>(mA, PACKED ? mB[k & 1] : mA, J, nt - 1, on_side ? cnt_side : cnt_main, q));
    if (PACKED)   // B of phase 3
      EAR_LAUNCH(k_dup16, grid_for(ndup), 256, 0, q)(reinterpret_cast<const uint16_t *>(Pk), Np, Pdk);
    prof_end(s2, q, (nt - 1) * tile_ops);
    return EAR_OK;
  };
  const int p3kind = PACKED ? PK_FW_P3_16 : PK_FW_P3;
  ear_status_t s = nt > 0 ? pivot(0, st) : EAR_OK;
  for (int k = 0; k < nt && s == EAR_OK; ++k) {
    if (k == 4 && pc && pc->hopeless()) {   // rounds 0-3 (~4 ms at cfg4 sizes) cover the SSSP
      *hopeless = true;
      break;
    }
    TileJob J{D, ldd, k * TILE, PACKED ? 0 : k * TILE, k, nt, 0, MODE_UPPER, 1};
    const CUtensorMap &B = PACKED ? mB[k & 1] : mA;
    if (!lookahead || k + 1 == nt) {
      const int64_t nup = (int64_t)(nt - 1) * nt / 2;
      int s3 = prof_begin(p3kind, st);
      s = launch_tiles<F>(mA, B, J, nup, cnt_main, st);
      prof_end(s3, st, nup * tile_ops);
      if (s == EAR_OK && k + 1 < nt) s = pivot(k + 1, st);
      continue;
    }
    debug_gpu_delay(st);
    int s3 = prof_begin(p3kind, st);
    J.mode = MODE_CROSS;
    s = launch_tiles<F>(mA, B, J, nt - 1, cnt_main, st);
    prof_end(s3, st, (nt - 1) * tile_ops);
    if (s != EAR_OK) break;
    cudaError_t e = cudaEventRecord(ctx->ev_cross, st);
    debug_host_delay();
    if (e == cudaSuccess) e = cudaStreamWaitEvent(ctx->side, ctx->ev_cross, 0);
    if (e != cudaSuccess) { set_error("fw_single: %s", cudaGetErrorString(e)); s = EAR_ECUDA; break; }
    s = pivot(k + 1, ctx->side);
    e = cudaEventRecord(ctx->ev_pivot, ctx->side);   // recorded even after an error: the main stream waits for it
    if (s == EAR_OK && e != cudaSuccess) { set_error("fw_single: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
    J.mode = MODE_REST;
    const int64_t nrest = (int64_t)(nt - 2) * (nt - 1) / 2;
    int s4 = prof_begin(p3kind, st);
    if (s == EAR_OK) s = launch_tiles<F>(mA, B, J, nrest, cnt_main, st, lookahead_reserve<F>(nrest, nt - 1));
    prof_end(s4, st, nrest * tile_ops);
    e = cudaStreamWaitEvent(st, ctx->ev_pivot, 0);
    if (s == EAR_OK && e != cudaSuccess) { set_error("fw_single: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  }
  return s;
}

// The packed FW on a capped copy of D.  *done = false (D untouched) when a connected pair reached the
// cap (or no memory for the copy); the caller then runs the int32 FW.  Synchronises the stream once.
ear_status_t fw_single16(int32_t *D, int64_t ldd, int32_t Np, const int32_t *lab, int32_t n_real, bool *done,
                         cudaStream_t st, ear_plan_s *plan, FwCtx *ctx, int32_t *cnt) {
  *done = false;
  Scratch sc(st);
  uint16_t *D16 = nullptr;
  uint32_t *Pd = nullptr;   // two 128 x Np buffers (round parity)
  int32_t *bad = nullptr;
  if (!sc.get(&D16, (size_t)Np * Np) || !sc.get(&Pd, 2 * (size_t)TILE * Np) || !sc.get(&bad, 1))
    return EAR_OK;   // no room for the 16-bit copy: the int32 path runs
  {
    int c0 = prof_begin(PK_FW16_CONV, st);
    EAR_LAUNCH(k_to16, grid_for((int64_t)Np * (Np / 4)), 256, 0, st)(D, ldd, D16, Np);
    prof_end(c0, st, 0);
  }
  // Cap precheck, overlapped with rounds 0-3: the exact distance row of reduced vertex 0 by one
  // single-source SSSP on a helper stream; its eccentricity is a lower bound on the largest finite
  // distance, so when it already reaches the cap the packed FW is abandoned after round 3 instead of
  // running to the end and being thrown away (cfg5: diameter ~42.8k).  Vertex 0 sits at a corner of the
  // spatially coherent labellings, so its eccentricity is close to the diameter.
  Precheck pc;
  pc.start(plan, Np, n_real, Np / TILE, ctx->h_word);
  bool hopeless = false;
  ear_status_t s = fw_single_sched<Frag16>(D16, Np, Np, Pd, ctx, cnt, st, &pc, &hopeless);
  if (s != EAR_OK) cudaStreamWaitEvent(st, ctx->ev_pivot, 0);   // never leave side work behind the frees
  pc.finish();
  if (s != EAR_OK) return s;
  if (hopeless) {
    prof_fw16_precheck();
    return EAR_OK;
  }
  int32_t h_bad = 1;
  int c1 = prof_begin(PK_FW16_CONV, st);
  EAR_CUDA_TRY(dev_memset(bad, 0, sizeof(int32_t), st));
  EAR_LAUNCH(k_check16, grid_for((int64_t)Np * (Np / 8)), 256, 0, st)(D16, Np, lab, n_real, bad);
  prof_end(c1, st, 0);
  {
    Readback rb(st);
    cudaError_t e = rb.get(&h_bad, bad, sizeof(int32_t));
    if (e == cudaSuccess) e = rb.sync();
    if (e != cudaSuccess) { set_error("fw_single16: %s", cudaGetErrorString(e)); return EAR_ECUDA; }
  }
  if (h_bad == 0) {
    int c2 = prof_begin(PK_FW16_CONV, st);
    EAR_LAUNCH(k_from16, grid_for((int64_t)Np * (Np / 4)), 256, 0, st)(D16, Np, D, ldd);
    prof_end(c2, st, 0);
    *done = true;
  }
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// ============================================================================== row-block sharding
// Symmetric row-block sharding.  Tile rows are dealt to ranks in a zig-zag (rows r and 2P-1-r of every
// group of 2P), so the UPPER tiles (ti, tj >= ti) -- the only authoritative ones -- balance across
// ranks; rank r stores its owned tile rows (ascending) as 128-row blocks.  Round k's pivot chain:
//   1. every rank copies its pieces of the pivot row block into L[k&1] (tile (k, j >= k) from the owner
//      of row k, tiles (i < k, k) transposed from the owners of rows i);
//   2. the owner of row k closes the pivot tile (phase 1) and pushes it into every peer's L[k&1];
//   3. every rank applies phase 2 to ITS pieces only (MODE_PIECES, one product against the closed tile);
//   4. every rank pushes its updated pieces into every rank's stage[k%3] and raises its flag -- the
//      per-round broadcast: each rank receives exactly the rest of the pivot row block, once;
//   5. once all flags are up, stage[k%3] is the complete updated block (packed: duplicated into the
//      B operand), and each rank copies its pieces back into its storage.
// Phase 3: every rank updates its owned upper tiles outside row/column k, both operands from stage.
// Per-rank min-plus work is (N_r^3 / 2) / P: the single-GPU symmetric halving survives the sharding.
// Buffer reuse is safe by the flag chain: a rank pushes round k+1's pieces only after it has every
// rank's round-k pieces, which each peer sends only after its own round k-1 phase 3 -- so a stage
// buffer is rewritten three rounds after its last reader, an L buffer two.
std::vector<int32_t> shard_rows_of(int32_t nt, int32_t P, int32_t rank) {
  std::vector<int32_t> rows;
  for (int32_t ti = 0; ti < nt; ++ti) {
    const int32_t o = ti % (2 * P);
    if ((o < P ? o : 2 * P - 1 - o) == rank) rows.push_back(ti);
  }
  return rows;
}

int zz_owner(int32_t ti, int32_t P) {
  const int32_t o = ti % (2 * P);
  return o < P ? o : 2 * P - 1 - o;
}

struct Shard {
  int32_t *S = nullptr;        // owned storage: nown x 128 rows x ldd (int32)
  int64_t ldd = 0;
  int32_t Np = 0, nt = 0, P = 1, rank = 0, nown = 0;
  std::vector<int32_t> rows;
  int32_t *d_rows = nullptr;
  int64_t *d_pre = nullptr;
  void pieces(int k, int *posk, int *mk, int *posk1 = nullptr) const {
    *posk = -1;
    *mk = 0;
    if (posk1) *posk1 = -1;
    for (int32_t r = 0; r < nown; ++r) {
      if (rows[r] < k) ++*mk;
      if (rows[r] == k) *posk = r;
      if (posk1 && rows[r] == k + 1) *posk1 = r;
    }
  }
};

ear_status_t shard_setup(Shard *sh, int32_t *S, int64_t ldd, int32_t Np, int32_t P, int32_t rank, Scratch &sc) {
  sh->S = S; sh->ldd = ldd; sh->Np = Np; sh->nt = Np / TILE; sh->P = P; sh->rank = rank;
  sh->rows = shard_rows_of(sh->nt, P, rank);
  sh->nown = (int32_t)sh->rows.size();
  std::vector<int64_t> pre(sh->nown + 1, 0);
  for (int32_t r = 0; r < sh->nown; ++r) pre[r + 1] = pre[r] + (sh->nt - sh->rows[r]);
  if (!sc.get(&sh->d_rows, sh->nown) || !sc.get(&sh->d_pre, sh->nown + 1)) {
    set_error("fw: out of device memory (shard tables)");
    return EAR_ENOMEM;
  }
  if (sh->nown > 0) {
    EAR_CUDA_TRY(cudaMemcpyAsync(sh->d_rows, sh->rows.data(), sizeof(int32_t) * sh->nown, cudaMemcpyHostToDevice, sc.st));
    EAR_CUDA_TRY(cudaMemcpyAsync(sh->d_pre, pre.data(), sizeof(int64_t) * (sh->nown + 1), cudaMemcpyHostToDevice, sc.st));
    EAR_CUDA_TRY(cudaStreamSynchronize(sc.st));   // host vectors are about to go out of scope
  }
  return EAR_OK;
}

// The sharded schedule for element policy F.  `sh` are the shards this process runs: one (its rank) with
// a communicator, or P virtual ranks sharing the buffers on one device (comm == nullptr: the pushes then
// land in the one shared stage and no flags are needed -- the same kernels and data movement otherwise).
// Stor[r]: shard r's storage in F's element type (int32: sh[r]->S itself; packed: a narrowed copy), all
// with leading dimension lds.  `solo` (rank timing): one rank's device work with the other ranks absent
// -- no waits, no pushes to peers, garbage data.
template <class F>
ear_status_t fw_sharded_sched(std::vector<Shard *> &sh, std::vector<typename F::E *> &Stor, int64_t lds, int32_t Np,
                              ear_comm_s *comm, FwCtx *ctx, int32_t *cnt, cudaStream_t st, Precheck *pc,
                              bool *hopeless, bool solo) {
  constexpr bool PACKED = sizeof(typename F::E) == 2;
  using E = typename F::E;
  const int nt = Np / TILE;
  const int P = sh[0]->P;
  const size_t R = sh.size();
  const int64_t nblk = (int64_t)TILE * Np;
  const bool lookahead = env_int("EAR_FW_LOOKAHEAD", 1) != 0;
  const double tile_ops = (double)TILE * TILE * TILE;
  *hopeless = false;
  Scratch sc(st);
  E *L[2] = {}, *stage[3] = {};
  uint32_t *Ld = nullptr, *Pd = nullptr;
  const bool real = comm && !solo;   // flags and pushes into the peers' windows
  if (real) {
    for (int b = 0; b < 2; ++b) L[b] = reinterpret_cast<E *>(comm_L(comm, comm->rank, b));
    for (int b = 0; b < 3; ++b) stage[b] = reinterpret_cast<E *>(comm_stage(comm, comm->rank, b));
  } else {
    bool ok = true;
    for (int b = 0; b < 2; ++b) ok = ok && sc.get(&L[b], nblk);
    for (int b = 0; b < 3; ++b) ok = ok && sc.get(&stage[b], nblk);
    if (!ok) { set_error("fw_sharded: out of device memory"); return EAR_ENOMEM; }
  }
  if (PACKED && (!sc.get(&Ld, nblk) || !sc.get(&Pd, 2 * nblk))) {
    set_error("fw_sharded: out of device memory");
    return EAR_ENOMEM;
  }
  CUtensorMap mL[2], mS[3], mLd, mPd[2];
  for (int b = 0; b < 2; ++b) EAR_TRY(make_map(&mL[b], (int)sizeof(E), L[b], TILE, Np, Np, F::KC));
  for (int b = 0; b < 3; ++b) EAR_TRY(make_map(&mS[b], (int)sizeof(E), stage[b], TILE, Np, Np, F::KC));
  if (PACKED) {
    EAR_TRY(make_map(&mLd, 4, Ld, TILE, Np, Np, F::KC));
    for (int b = 0; b < 2; ++b) EAR_TRY(make_map(&mPd[b], 4, Pd + b * nblk, TILE, Np, Np, F::KC));
  }
  int32_t *cnt_main = cnt, *cnt_side = cnt + 2, *cnt_push = cnt + 4;
  // destinations of this rank's pushes: every rank's stage[b] (comm), the shared one otherwise
  auto stage_dsts = [&](int b) {
    PeerPtrs d{};
    if (real) {
      d.n = comm->nranks;
      for (int p = 0; p < comm->nranks; ++p) d.p[p] = comm_stage(comm, p, b);
    } else {
      d.n = 1;
      d.p[0] = reinterpret_cast<char *>(stage[b]);
    }
    return d;
  };
  // round k's pivot chain on stream q
  auto chain = [&](int k, cudaStream_t q) -> ear_status_t {
    const bool on_side = q != st;
    const int b = k & 1, s3 = k % 3;
    int32_t *cq = on_side ? cnt_side : cnt_main;
    for (size_t r = 0; r < R; ++r) {
      int posk, mk;
      sh[r]->pieces(k, &posk, &mk);
      const int np = (posk >= 0 ? nt - k : 0) + mk;
      if (np > 0)
        EAR_LAUNCH(k_prow_xfer<E>, dim3(16, np), 256, 0, q)(Stor[r], lds, sh[r]->d_rows, k, nt, posk, L[b], Np, 0);
    }
    const int owner = zz_owner(k, P);
    const bool mine = real ? comm->rank == owner : true;   // emulated / solo: the owner is local
    int s1 = prof_begin(on_side ? PK_FW_SIDE_P1 : PK_FW_P1, q);
    if (mine) {
      if (PACKED)
        EAR_LAUNCH(k_fw_phase1_16, 1, NT, 0, q)(reinterpret_cast<uint16_t *>(L[b]) + (int64_t)k * TILE, Np);
      else
        EAR_LAUNCH(k_fw_phase1, 1, NT, 0, q)(reinterpret_cast<int32_t *>(L[b]) + (int64_t)k * TILE, Np);
    }
    prof_end(s1, q, mine ? tile_ops : 0.0);
    if (real && P > 1) {   // the closed pivot tile from its owner into every peer's L[b]
      int sc1 = prof_begin(PK_COMM, q);
      const uint64_t v = ++comm->seq_tile;
      if (mine) {
        PeerPtrs d{}, f{};
        for (int p = 0; p < P; ++p)
          if (p != comm->rank) {
            d.p[d.n] = comm_L(comm, p, b);
            f.p[f.n] = comm->peer[p];
            ++d.n;
            ++f.n;
          }
        // one "piece": column block k of the owner's L (posk = 0 with nt = k + 1 selects just it)
        EAR_LAUNCH(k_push_pieces<E>, dim3(1, 4), 256, 0, q)(L[b], Np, k, k + 1, 0, 0, sh[0]->d_rows, d, cnt_push, f,
                                                            SLOT_TILE + comm->rank, v);
      } else {
        EAR_TRY(comm_wait_one(comm, SLOT_TILE + owner, v, q));
      }
      prof_end(sc1, q, 0);
    }
    int s2 = prof_begin(on_side ? PK_FW_SIDE_P2 : PK_FW_P2, q);
    if (PACKED) EAR_LAUNCH(k_dup16, grid_for(nblk / 4), 256, 0, q)(reinterpret_cast<uint16_t *>(L[b]), Np, Ld);
    double p2 = 0;
    for (size_t r = 0; r < R; ++r) {
      int posk, mk;
      sh[r]->pieces(k, &posk, &mk);
      const int64_t n2 = mk + (posk >= 0 ? nt - 1 - k : 0);
      if (n2 == 0) continue;
      TileJob J2{L[b], Np, 0, 0, k, nt, k, MODE_PIECES, 0, 0, sh[r]->d_rows, sh[r]->d_pre, sh[r]->nown, mk, posk, -1};
      EAR_TRY(launch_tiles<F>(mL[b], PACKED ? mLd : mL[b], J2, n2, cq, q));
      p2 += (double)n2 * tile_ops;
    }
    prof_end(s2, q, p2);
    int sc2 = prof_begin(PK_COMM, q);
    const uint64_t vp = real ? ++comm->seq_pieces : 0;
    for (size_t r = 0; r < R; ++r) {
      int posk, mk;
      sh[r]->pieces(k, &posk, &mk);
      const int np = (posk >= 0 ? nt - k : 0) + mk;
      if (np == 0 && !real) continue;
      const PeerPtrs f = real ? comm_flags_all(comm) : PeerPtrs{};
      EAR_LAUNCH(k_push_pieces<E>, dim3(std::max(np, 1), 4), 256, 0, q)(L[b], Np, k, nt, posk, mk, sh[r]->d_rows,
                                                                        stage_dsts(s3), real ? cnt_push : nullptr, f,
                                                                        SLOT_PIECES + (real ? comm->rank : 0), vp);
    }
    if (real) EAR_TRY(comm_wait(comm, SLOT_PIECES, vp, q));
    prof_end(sc2, q, 0);
    if (PACKED)
      EAR_LAUNCH(k_dup16, grid_for(nblk / 4), 256, 0, q)(reinterpret_cast<uint16_t *>(stage[s3]), Np, Pd + b * nblk);
    for (size_t r = 0; r < R; ++r) {
      int posk, mk;
      sh[r]->pieces(k, &posk, &mk);
      const int np = (posk >= 0 ? nt - k : 0) + mk;
      if (np > 0)
        EAR_LAUNCH(k_prow_xfer<E>, dim3(16, np), 256, 0, q)(Stor[r], lds, sh[r]->d_rows, k, nt, posk, stage[s3], Np, 1);
    }
    return EAR_OK;
  };
  auto phase3 = [&](int k, int mode, cudaStream_t q, int reserve) -> ear_status_t {
    const CUtensorMap &A = mS[k % 3], &B = PACKED ? mPd[k & 1] : mS[k % 3];
    for (size_t r = 0; r < R; ++r) {
      const Shard &s = *sh[r];
      int posk, mk, posk1;
      s.pieces(k, &posk, &mk, &posk1);
      int64_t total = 0;
      for (int32_t i = 0; i < s.nown; ++i) {
        const int32_t ti = s.rows[i];
        const int64_t all = ti == k ? 0 : (nt - ti) - (ti < k ? 1 : 0);
        const int64_t cross = (ti == k + 1 ? nt - ti : 0) + (ti < k ? 1 : 0);
        total += mode == MODE_LIST ? all : mode == MODE_LIST_CROSS ? cross : all - cross;
      }
      if (total == 0) continue;
      const int res = reserve < 0 ? lookahead_reserve<F>(total, (nt - 1 + P - 1) / P) : reserve;
      TileJob J{Stor[r], lds, 0, 0, k, nt, 0, mode, 0, 0, s.d_rows, s.d_pre, s.nown, mk, posk, posk1};
      int s3 = prof_begin(PACKED ? PK_FW_P3_16 : PK_FW_P3, q);
      EAR_TRY(launch_tiles<F>(A, B, J, total, cnt_main, q, res));
      prof_end(s3, q, (double)total * tile_ops);
    }
    return EAR_OK;
  };
  ear_status_t s = chain(0, st);
  for (int k = 0; k < nt && s == EAR_OK; ++k) {
    if (k == 4 && pc && pc->hopeless()) {
      *hopeless = true;
      break;
    }
    if (!lookahead || k + 1 == nt) {
      s = phase3(k, MODE_LIST, st, 0);
      if (s == EAR_OK && k + 1 < nt) s = chain(k + 1, st);
      continue;
    }
    debug_gpu_delay(st);
    s = phase3(k, MODE_LIST_CROSS, st, 0);
    if (s != EAR_OK) break;
    cudaError_t e = cudaEventRecord(ctx->ev_cross, st);
    debug_host_delay();
    if (e == cudaSuccess) e = cudaStreamWaitEvent(ctx->side, ctx->ev_cross, 0);
    if (e != cudaSuccess) { set_error("fw_sharded: %s", cudaGetErrorString(e)); s = EAR_ECUDA; break; }
    s = chain(k + 1, ctx->side);
    e = cudaEventRecord(ctx->ev_pivot, ctx->side);   // recorded even after an error: the main stream waits for it
    if (s == EAR_OK && e != cudaSuccess) { set_error("fw_sharded: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
    if (s == EAR_OK) s = phase3(k, MODE_LIST_REST, st, -1);
    e = cudaStreamWaitEvent(st, ctx->ev_pivot, 0);
    if (s == EAR_OK && e != cudaSuccess) { set_error("fw_sharded: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  }
  if (s != EAR_OK) cudaStreamWaitEvent(st, ctx->ev_pivot, 0);
  return s;
}

// Sharded FW over the shards `sh` (one rank with comm, or emulated ranks): the packed schedule first
// (allow16; exact unless a connected pair reaches the cap -- checked over every rank's upper tiles and
// agreed through the CHECK flags), the int32 schedule on the untouched int32 storage otherwise.
ear_status_t fw_sharded_run(std::vector<Shard *> &sh, int32_t Np, ear_comm_s *comm, const int32_t *lab, int32_t n_real,
                            bool allow16, cudaStream_t st, ear_plan_s *plan, bool solo, bool *used16) {
  *used16 = false;
  const int nt = Np / TILE;
  const size_t R = sh.size();
  FwCtx *ctx = nullptr;
  EAR_TRY(ctx_acquire(&ctx));
  CtxLease lease{ctx};
  Scratch sc(st);
  int32_t *cnt = nullptr;
  if (!sc.get(&cnt, 8)) { set_error("fw_sharded: out of device memory"); return EAR_ENOMEM; }
  EAR_CUDA_TRY(dev_memset(cnt, 0, 8 * sizeof(int32_t), st));
  if (comm && !solo) EAR_TRY(comm_barrier(comm, st));   // every peer is done with the previous call's buffers
  if (allow16 && nt >= 2) {
    std::vector<uint16_t *> S16(R, nullptr);
    int32_t *flag = nullptr;
    bool ok = sc.get(&flag, 1);
    for (size_t r = 0; r < R && ok; ++r) ok = sc.get(&S16[r], (size_t)std::max(sh[r]->nown, 1) * TILE * Np);
    if (ok) {
      int c0 = prof_begin(PK_FW16_CONV, st);
      for (size_t r = 0; r < R; ++r)
        if (sh[r]->nown > 0)
          EAR_LAUNCH(k_to16r, grid_for((int64_t)sh[r]->nown * TILE * (Np / 4)), 256, 0, st)(
              sh[r]->S, sh[r]->ldd, S16[r], Np, (int64_t)sh[r]->nown * TILE, Np);
      prof_end(c0, st, 0);
      Precheck pc;   // as fw_single16's; every rank decides the same
      if (!solo) pc.start(plan, Np, n_real, nt, ctx->h_word);
      bool hopeless = false;
      ear_status_t s = fw_sharded_sched<Frag16>(sh, S16, Np, Np, comm, ctx, cnt, st, &pc, &hopeless, solo);
      pc.finish();
      EAR_TRY(s);
      if (hopeless) {
        prof_fw16_precheck();
      } else if (solo) {
        *used16 = true;
        return EAR_OK;   // rank timing: no check, no result
      } else {
        int c1 = prof_begin(PK_FW16_CONV, st);
        EAR_CUDA_TRY(dev_memset(flag, 0, sizeof(int32_t), st));
        for (size_t r = 0; r < R; ++r)
          if (sh[r]->nown > 0)
            EAR_LAUNCH(k_check16_list, grid_for((int64_t)sh[r]->nown * TILE * (Np / 8)), 256, 0, st)(
                S16[r], Np, sh[r]->d_rows, sh[r]->nown, Np, lab, n_real, flag);
        prof_end(c1, st, 0);
        if (comm && comm->nranks > 1) {   // OR of every rank's bit
          const uint64_t v = ++comm->seq_check;
          EAR_LAUNCH(k_check_push, 1, 32, 0, st)(flag, comm_flags_all(comm), SLOT_CHECK + comm->rank, v);
          EAR_TRY(comm_wait(comm, SLOT_CHECK, v << 1, st));
          EAR_LAUNCH(k_check_fold, 1, 32, 0, st)(reinterpret_cast<const uint64_t *>(comm->win) + SLOT_CHECK,
                                                 comm->nranks, flag);
        }
        int32_t h_flag = -1;
        Readback rb(st);
        cudaError_t e = rb.get(&h_flag, flag, sizeof(int32_t));
        if (e == cudaSuccess) e = rb.sync();
        if (e != cudaSuccess) { set_error("fw_sharded: %s", cudaGetErrorString(e)); return EAR_ECUDA; }
        if (h_flag == 0) {
          int c2 = prof_begin(PK_FW16_CONV, st);
          for (size_t r = 0; r < R; ++r)
            if (sh[r]->nown > 0)
              EAR_LAUNCH(k_from16r, grid_for((int64_t)sh[r]->nown * TILE * (Np / 4)), 256, 0, st)(
                  S16[r], Np, sh[r]->S, sh[r]->ldd, (int64_t)sh[r]->nown * TILE, Np);
          prof_end(c2, st, 0);
          *used16 = true;
          return EAR_OK;
        }
      }
    } else {
      cudaGetLastError();   // no room for the 16-bit copies: the int32 schedule runs
    }
  }
  std::vector<int32_t *> S32(R);
  for (size_t r = 0; r < R; ++r) S32[r] = sh[r]->S;
  bool hopeless = false;
  // every shard's storage has the same leading dimension (the callers allocate them alike)
  return fw_sharded_sched<Frag32>(sh, S32, sh[0]->ldd, Np, comm, ctx, cnt, st, nullptr, &hopeless, solo);
}

}  // namespace

// ============================================================================== internal API
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

// Single GPU: full symmetric D (Np x Np).  With allow16 the packed FW runs first on a copy and its
// result is kept when no connected pair (labels lab over [0, n_real), or one component when lab is
// NULL) reached the cap; otherwise, or without allow16, the int32 schedule runs on D.
ear_status_t fw_single(int32_t *D, int64_t ldd, int32_t Np, cudaStream_t st, const int32_t *lab, int32_t n_real,
                       bool allow16, ear_plan_s *plan) {
  NvtxRange nvtx_("ear: blocked FW");
  FwCtx *ctx = nullptr;
  EAR_TRY(ctx_acquire(&ctx));
  CtxLease lease{ctx};
  Scratch sc(st);
  int32_t *cnt = nullptr;   // tile counter pairs: main stream, side stream
  if (!sc.get(&cnt, 4)) { set_error("fw_single: out of device memory"); return EAR_ENOMEM; }
  EAR_CUDA_TRY(dev_memset(cnt, 0, 4 * sizeof(int32_t), st));
  if (allow16 && Np >= 2 * TILE) {
    bool done = false;
    EAR_TRY(fw_single16(D, ldd, Np, lab, n_real, &done, st, plan, ctx, cnt));
    prof_fw16(done);
    if (done) return EAR_OK;
  }
  bool hopeless = false;
  ear_status_t s = fw_single_sched<Frag32>(D, ldd, Np, nullptr, ctx, cnt, st, nullptr, &hopeless);
  if (s != EAR_OK) cudaStreamWaitEvent(st, ctx->ev_pivot, 0);
  EAR_TRY(s);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

std::vector<int32_t> shard_rows(int32_t nt, int32_t P, int32_t rank) { return shard_rows_of(nt, P, rank); }

int32_t shard_nown(int32_t nt, int32_t P, int32_t rank) { return (int32_t)shard_rows_of(nt, P, rank).size(); }

ear_status_t shard_rows_device(int32_t nt, int32_t P, int32_t rank, int32_t **d_rows, int32_t *nown, cudaStream_t st) {
  std::vector<int32_t> rows = shard_rows_of(nt, P, rank);
  *nown = (int32_t)rows.size();
  EAR_CUDA_TRY(cudaMallocAsync((void **)d_rows, sizeof(int32_t) * std::max<size_t>(rows.size(), 1), st));
  if (!rows.empty()) {
    EAR_CUDA_TRY(cudaMemcpyAsync(*d_rows, rows.data(), sizeof(int32_t) * rows.size(), cudaMemcpyHostToDevice, st));
    EAR_CUDA_TRY(cudaStreamSynchronize(st));
  }
  return EAR_OK;
}

// this rank's owned-row storage inside its window (collective: reserves the window for Np)
ear_status_t fw_shard_buffer(ear_comm_s *comm, int32_t Np, cudaStream_t st, int32_t **S) {
  const int32_t nown = shard_nown(Np / TILE, comm->nranks, comm->rank);
  EAR_TRY(comm_reserve(comm, Np, nown, st));
  *S = comm_region(comm, comm->rank);
  return EAR_OK;
}

// Sharded FW on a rank's owned int32 rows S (ld ldd >= Np): packed schedule first (allow16), int32
// otherwise.  Collective over the communicator's ranks.
ear_status_t fw_sharded_auto(int32_t *S, int64_t ldd, int32_t Np, ear_comm_s *comm, const int32_t *lab,
                             int32_t n_real, bool allow16, cudaStream_t st, ear_plan_s *plan) {
  EAR_TRY(comm_reserve(comm, Np, shard_nown(Np / TILE, comm->nranks, comm->rank), st));
  Scratch sc(st);
  Shard sh;
  EAR_TRY(shard_setup(&sh, S, ldd, Np, comm->nranks, comm->rank, sc));
  std::vector<Shard *> v{&sh};
  bool used16 = false;
  EAR_TRY(fw_sharded_run(v, Np, comm, lab, n_real, allow16, st, plan, false, &used16));
  if (allow16 && Np >= 2 * TILE) prof_fw16(used16);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// One rank's device work of a P-rank sharded FW, without the other ranks and the exchange
// (apsp_reduced_rank_timing: per-rank compute scaling measured on one GPU); packed unless fw32.
ear_status_t fw_rank_timing(const ear_plan_s *plan, int32_t Np, int32_t P, int32_t rank, bool fw32, cudaStream_t st) {
  Scratch sc(st);
  const size_t nown = shard_rows_of(Np / TILE, P, rank).size();
  int32_t *S = nullptr;
  if (!sc.get(&S, std::max<size_t>(nown, 1) * TILE * Np)) { set_error("rank timing: out of memory"); return EAR_ENOMEM; }
  Shard sh;
  EAR_TRY(shard_setup(&sh, S, Np, Np, P, rank, sc));
  for (int32_t lr = 0; lr < sh.nown; ++lr)
    EAR_TRY(fw_init_D(plan, S + (int64_t)lr * TILE * Np, Np, Np, sh.rows[lr] * TILE, TILE, st));
  std::vector<Shard *> v{&sh};
  bool used16 = false;
  return fw_sharded_run(v, Np, nullptr, nullptr, plan->n_reduced, !fw32, st, nullptr, true, &used16);
}

// Full D (Np x Np, ldf) from every rank's owned upper tiles: the rank's storage S goes into its window
// region (unless it is already there), a barrier, then every rank reads every tile from the window of
// its owner (the mirror of the lower triangle fused into the same pass), then a barrier so no rank
// rewrites its region while a peer still reads it.  Collective.
ear_status_t fw_sharded_gather(const int32_t *S, int64_t ldd, int32_t Np, int32_t *Df, int64_t ldf, ear_comm_s *comm,
                               cudaStream_t st) {
  const int32_t nt = Np / TILE, P = comm->nranks;
  const int32_t nown = shard_nown(nt, P, comm->rank);
  EAR_TRY(comm_reserve(comm, Np, nown, st));
  int32_t *reg = comm_region(comm, comm->rank);
  if (S != reg && nown > 0)
    EAR_CUDA_TRY(cudaMemcpy2DAsync(reg, sizeof(int32_t) * Np, S, sizeof(int32_t) * ldd, sizeof(int32_t) * Np,
                                   (size_t)nown * TILE, cudaMemcpyDeviceToDevice, st));
  int sc = prof_begin(PK_COMM, st);
  EAR_TRY(comm_barrier(comm, st));
  PeerPtrs regions{};
  regions.n = P;
  for (int p = 0; p < P; ++p) regions.p[p] = reinterpret_cast<char *>(comm_region(comm, p));
  if (nt > 0) EAR_LAUNCH(k_gather_pull, dim3(nt, nt), 256, 0, st)(regions, P, Np, Df, ldf);
  EAR_TRY(comm_barrier(comm, st));
  prof_end(sc, st, 0);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// The same schedule for P ranks emulated in one process on one device (tests of the multi-GPU path on
// one GPU): every virtual rank has its own owned storage, they share the pivot-row buffers (their pieces
// are disjoint), and the ranks' upper tiles are scattered into D.
ear_status_t fw_sharded_emulated(ear_plan_s *plan, int32_t *D, int64_t ldd, int32_t Np, int32_t P, cudaStream_t st) {
  const int nt = Np / TILE;
  Scratch sc(st);
  std::vector<Shard> sh(P);
  for (int r = 0; r < P; ++r) {
    const size_t nown = shard_rows_of(nt, P, r).size();
    int32_t *S = nullptr;
    if (!sc.get(&S, std::max<size_t>(nown, 1) * TILE * Np)) { set_error("emulated: out of memory"); return EAR_ENOMEM; }
    EAR_TRY(shard_setup(&sh[r], S, Np, Np, P, r, sc));
    for (int32_t lr = 0; lr < sh[r].nown; ++lr)
      EAR_TRY(fw_init_D(plan, S + (int64_t)lr * TILE * Np, Np, Np, sh[r].rows[lr] * TILE, TILE, st));
  }
  const bool allow16 = !(plan->flags & EAR_FLAG_FW32);
  const int32_t *lab = nullptr;
  if (allow16) EAR_TRY(reduced_labels(plan, Np, st, &lab));
  std::vector<Shard *> v;
  for (int r = 0; r < P; ++r) v.push_back(&sh[r]);
  bool used16 = false;
  EAR_TRY(fw_sharded_run(v, Np, nullptr, lab, plan->n_reduced, allow16, st, plan, false, &used16));
  if (allow16 && Np >= 2 * TILE) prof_fw16(used16);
  for (int r = 0; r < P; ++r) {
    if (sh[r].nown == 0) continue;
    dim3 g(16, nt, sh[r].nown);
    EAR_LAUNCH(k_scatter_upper, g, 256, 0, st)(sh[r].S, sh[r].ldd, sh[r].d_rows, D, ldd);
  }
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
    EAR_CUDA_TRY(cudaMallocAsync((void **)&changed, 4 * sizeof(int32_t), st));
    p->cc_np = Np;
    ear_status_t s = EAR_OK;
    {
      int per_sm = 0;
      EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_cc_coop, 256, 0));
      const int64_t work = std::max<int64_t>(Np, p->n_redges);
      const int g = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(work, 256), (int64_t)per_sm * num_sms()));
      const int32_t *ru = p->re_u, *rv = p->re_v;
      int64_t E = p->n_redges;
      int32_t *lab = p->cc, nn = Np;
      void *args[] = {(void *)&ru, (void *)&rv, (void *)&E, (void *)&lab, (void *)&nn, (void *)&changed};
      EAR_CUDA_TRY(dev_memset(changed, 0, 4 * sizeof(int32_t), st));
      count_launch();
      cudaError_t e = cudaLaunchCooperativeKernel((const void *)k_cc_coop, g, 256, args, 0, st);
      if (e != cudaSuccess) { set_error("reduced_labels: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
    }
    cudaFreeAsync(changed, st);
    EAR_TRY(s);
  }
  *out = p->cc;
  return EAR_OK;
}

}  // namespace ear
