// Phase II by REGIONS: a vertex partition of G^r composed through the region boundaries
// (EAR_FLAG_PART).  This is sec. 2.2's composition through articulation points (P:129-131,
// "d(n1, n2) = d(n1, a1) + d(a1, a2) + d(a2, n2)") with the one-vertex separators replaced by the
// boundary SETS of small regions -- reading C24 in DESIGN.md.
//
// Let the vertices of G^r be partitioned into connected regions R_1..R_K, and B_i be the vertices of
// R_i with a neighbour outside R_i (the boundary), B their union.  d_i is the distance inside the
// subgraph induced by R_i, d the distance in G^r.  A shortest u-v path (u in R_i) either stays inside
// R_i, or leaves it for the first time from some b in B_i, so
//     d(u, v) = min( [v in R_i] d_i(u, v),  min_{b in B_i} d_i(u, b) + d(b, v) )            (1)
// (every term is the length of a walk, hence >= d(u, v), and the first-exit term is exact).  The same
// argument on the last entry into R_j gives, for b in B and v in R_j,
//     d(b, v) = min_{b' in B_j} d(b, b') + d_j(b', v)                                         (2)
// and the distances between boundary vertices are those of the boundary graph on B with the cliques
// d_i(b, b') (b, b' in B_i) and the arcs of G^r that join two regions:
//     d(b, b') = FW over B                                                                     (3)
// The kernels, in that order:
//   * k_partition (one cooperative launch): regions = Voronoi cells of a multi-source hop BFS (seeds
//     every PSEED ids plus one vertex per connected component, ties to the smaller seed id), cells larger
//     than PCAP split again inside themselves with denser seeds -- label-independent up to the seeds;
//   * CUB radix sort of (region, boundary-first) keys -> every region's members contiguous, its
//     boundary first; region / boundary offsets by scans;
//   * k_region_fw: d_i for every region, one CTA per region, the PCAP x PCAP matrix in registers (8 x 16
//     entries per thread as packed u16x2, one VIADDMNMX.U16x2 per two min-plus, capped at 0x7FFF);
//   * (3): the boundary graph H (cliques + joining arcs) solved by this same route when |B| >= PREC_MIN
//     (nested), else densely by k_fw64 (one cooperative launch of a 64-tile FW, capped u16), with the
//     blocked FW of fw.cu (int32) when a connected pair reaches the cap;
//   * k_region_prod<false>: (2) for every region j and every boundary column tile -> DBVt[v][b] = d(b, v),
//     then k_transpose16 -> DBV[b][v];
//   * k_region_prod<true>: (1) for every region i and every column tile of D -> the u16 rows of D
//     (k_region_mp: both products for regions whose boundary exceeds 32).
// The two products are min-plus products with the region's boundary as the inner dimension
// (K = |B_i|, ~10-40 on the paper's sparse graphs): dense work on the ALU pipe at N_r^2 * mean|B_i|
// min-plus, against the per-source SSSP's N_r * M_r relaxations in hundreds of dependent rounds.
//
// Exactness: all distances are integers; the u16 lanes of VIADDMNMX.U16x2 add without saturation, so
// each product runs only when none of its sums of two operands of one component can reach 0x10000:
// Lmax + max(dB) < 0xFFFF for (2), Lmax + max(DBV) < 0xFFFF for (1) (Lmax the largest d_i; the maxima
// over finite entries, taken on the device and checked by the product kernels themselves).  Sums that
// involve INF (0xFFFF, other components) wrap, but they only reach entries of pairs in different
// components, which the last product overwrites with INF.  Otherwise *applied = false and the caller
// runs another Phase II route.
#include <cooperative_groups.h>
#include <cub/cub.cuh>

#include <algorithm>
#include <chrono>
#include <climits>
#include <cstdlib>

#include "common.cuh"

struct ear_part_s {
  int32_t K = 0, NB = 0, NBp = 0, passes = 0, max_region = 0, max_bnd = 0, multi = 0;
  double sum_rb = 0;                 // sum over regions of |R_i| |B_i| (product work / N_r)
  int32_t *reg = nullptr;            // [nr] region of v
  int32_t *loc = nullptr;            // [nr] index of v inside its region (boundary first)
  int32_t *perm = nullptr;           // [nr] members of region i at perm[roff[i] .. roff[i+1])
  int32_t *roff = nullptr;           // [K+1]
  int32_t *bcnt = nullptr;           // [K] |B_i|
  int32_t *boff = nullptr;           // [K] first global boundary index of region i
  int32_t *rcomp = nullptr;          // [K] connected component (cc label) of region i
  int32_t *bvert = nullptr;          // [NB] vertex of global boundary index g
  int32_t *gidx = nullptr;           // [nr] global boundary index, -1 inside
  int32_t *big = nullptr;            // [nbig] regions with |B_i| > MP_KC (the general product kernel)
  int32_t nbig = 0;
  int2 *vrange = nullptr;            // [K] smallest / largest vertex id of region i
};

namespace ear {
ear_status_t sssp_prepare(ear_plan_s *p, cudaStream_t st);

// a graph as the region route reads it: CSR (both arc directions, parallel arcs merged), and connected-
// component labels that are the smallest vertex id of the component
struct GView {
  int32_t n;
  const int32_t *rowptr, *col, *w, *cc;
};

namespace {

constexpr int PCAP = 256;            // largest region: its d_i is one CTA's register file
constexpr int PSEED = 160;           // seed spacing (in vertex ids) of the first Voronoi pass
constexpr uint32_t PC16 = 0x7FFF;    // cap of the region FW (two capped values never wrap)
constexpr int FW_NT = 512;
constexpr int MP_NT = 256, MP_TC = 128, MP_KC = 32, MP_BS = MP_TC + 8;   // Bs row stride (u16): 4-way max
constexpr int PR_NT = 128, PR_MIN = 4;   // k_region_prod: 128 threads, 4 CTAs per SM (measured: 256 x 2 and 512 x 1 slower)
constexpr int NT = 256;
constexpr int PREC_MIN = 2048;      // a boundary graph this large is solved by regions again
constexpr int PREC_DEPTH = 2;       // ... down to this nesting depth (then by the blocked FW)
constexpr int FW64_MAX = 8192;      // dense boundary matrices up to this size: the 64-tile cooperative FW

int grid_n(int64_t n) { return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, NT), 148 * 16)); }

__device__ __forceinline__ uint32_t dup16(uint32_t x) { return x | (x << 16); }

__global__ void k_keys(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col, int32_t n,
                       const int32_t *__restrict__ lab, uint32_t *keys, int32_t *vals) {
  for (int32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
    const int32_t l = lab[v];
    bool bnd = false;
    for (int32_t a = rowptr[v], e = rowptr[v + 1]; a < e && !bnd; ++a) bnd = lab[col[a]] != l;
    keys[v] = ((uint32_t)l << 1) | (bnd ? 0u : 1u);
    vals[v] = v;
  }
}

__global__ void k_flags(const uint32_t *__restrict__ sk, int32_t n, int32_t *fstart, int32_t *fbnd) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    fstart[i] = (i == 0 || (sk[i] >> 1) != (sk[i - 1] >> 1)) ? 1 : 0;
    fbnd[i] = (sk[i] & 1u) ? 0 : 1;
  }
}

// rid = inclusive scan of fstart (region + 1), gpos = exclusive scan of fbnd
__global__ void k_fill(const int32_t *__restrict__ perm, const int32_t *__restrict__ fstart,
                       const int32_t *__restrict__ fbnd, const int32_t *__restrict__ rid,
                       const int32_t *__restrict__ gpos, const int32_t *__restrict__ cc, int32_t n, int32_t *reg,
                       int32_t *gidx, int32_t *roff, int32_t *boff, int32_t *bcnt, int32_t *rcomp, int32_t *bvert,
                       int32_t *tot) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t v = perm[i], r = rid[i] - 1;
    reg[v] = r;
    if (fstart[i]) {
      roff[r] = i;
      boff[r] = gpos[i];
      rcomp[r] = cc[v];
    }
    if (fbnd[i]) {
      gidx[v] = gpos[i];
      bvert[gpos[i]] = v;
      atomicAdd(&bcnt[r], 1);
    } else {
      gidx[v] = -1;
    }
    if (i == n - 1) {
      roff[r + 1] = n;
      tot[0] = r + 1;
      tot[1] = gpos[i] + fbnd[i];
    }
  }
}

__global__ void k_loc(const int32_t *__restrict__ perm, const int32_t *__restrict__ rid,
                      const int32_t *__restrict__ roff, int32_t n, int32_t *loc, int32_t *stats) {
  int mx = 0;
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t r = rid[i] - 1;
    loc[perm[i]] = i - roff[r];
    if (i + 1 == n || rid[i + 1] != rid[i]) mx = max(mx, i + 1 - roff[r]);
  }
  for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(stats, mx);
}

// d_i of region i (blockIdx.x): thread (rg, cg) holds rows rg*8..+8, columns cg*16..+16 as 8 x 8 packed
// pairs; round kk reads row kk (= column kk: d_i is symmetric) from a shared row buffer that the owners
// of row kk+1 refill after their update -- one barrier per round.  Capped at PC16 (exact below it).
__global__ void __launch_bounds__(FW_NT, 1)
    k_region_fw(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col, const int32_t *__restrict__ w,
                const int32_t *__restrict__ roff, const int32_t *__restrict__ perm, const int32_t *__restrict__ reg,
                const int32_t *__restrict__ loc, uint16_t *__restrict__ LR, int32_t *stats) {
  extern __shared__ __align__(16) uint16_t M[];   // PCAP x PCAP, then two row buffers
  uint16_t *rowbuf = M + PCAP * PCAP;
  __shared__ int s_max, s_over;
  const int i = blockIdx.x, tid = threadIdx.x;
  const int32_t r0 = roff[i], r = roff[i + 1] - r0, rp = (r + 7) & ~7;
  if (tid == 0) s_max = 0, s_over = 0;
  for (int e = tid; e < PCAP * PCAP / 2; e += FW_NT) {
    const int row = (2 * e) / PCAP, c = (2 * e) % PCAP;
    reinterpret_cast<uint32_t *>(M)[e] = (row == c ? 0u : PC16) | ((row == c + 1 ? 0u : PC16) << 16);
  }
  __syncthreads();
  int over = 0;
  for (int a = tid; a < r; a += FW_NT) {
    const int32_t v = perm[r0 + a];
    for (int32_t t = rowptr[v], e = rowptr[v + 1]; t < e; ++t) {
      const int32_t x = col[t];
      if (reg[x] != i) continue;
      const int32_t wt = w[t];
      if (wt >= (int32_t)PC16) over = 1;
      const int j = loc[x];
      const uint16_t ww = (uint16_t)min(wt, (int32_t)PC16);
      if (ww < M[a * PCAP + j]) M[a * PCAP + j] = ww;
    }
  }
  __syncthreads();
  const int rg = tid >> 4, cg = tid & 15;
  uint32_t c[8][8];
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const uint4 *src = reinterpret_cast<const uint4 *>(M + (rg * 8 + q) * PCAP + cg * 16);
    const uint4 x0 = src[0], x1 = src[1];
    c[q][0] = x0.x, c[q][1] = x0.y, c[q][2] = x0.z, c[q][3] = x0.w;
    c[q][4] = x1.x, c[q][5] = x1.y, c[q][6] = x1.z, c[q][7] = x1.w;
  }
  if (tid < PCAP / 8) reinterpret_cast<uint4 *>(rowbuf)[tid] = reinterpret_cast<const uint4 *>(M)[tid];
  __syncthreads();
  for (int kb = 0; kb < rp / 8; ++kb) {
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const int kk = kb * 8 + q;
      const uint16_t *rb = rowbuf + (kk & 1) * PCAP;
      const uint4 av = *reinterpret_cast<const uint4 *>(rb + rg * 8);
      const uint4 b0 = *reinterpret_cast<const uint4 *>(rb + cg * 16);
      const uint4 b1 = *reinterpret_cast<const uint4 *>(rb + cg * 16 + 8);
      const uint32_t aw[4] = {av.x, av.y, av.z, av.w};
      const uint32_t b[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
      for (int rr = 0; rr < 8; ++rr) {
        const uint32_t a = dup16((aw[rr >> 1] >> ((rr & 1) * 16)) & 0xFFFFu);
#pragma unroll
        for (int p = 0; p < 8; ++p) c[rr][p] = __viaddmin_u16x2(a, b[p], c[rr][p]);
      }
      const int nq = (q + 1) & 7;   // compile-time after unrolling
      if (kk + 1 < rp && rg == kb + (q == 7 ? 1 : 0)) {
        uint4 *dst = reinterpret_cast<uint4 *>(rowbuf + ((kk + 1) & 1) * PCAP + cg * 16);
        dst[0] = make_uint4(c[nq][0], c[nq][1], c[nq][2], c[nq][3]);
        dst[1] = make_uint4(c[nq][4], c[nq][5], c[nq][6], c[nq][7]);
      }
      __syncthreads();
    }
  }
  int mx = 0;
  uint16_t *out = LR + (size_t)i * PCAP * PCAP;
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const int row = rg * 8 + q;
    if (row >= rp) continue;
    uint4 *dst = reinterpret_cast<uint4 *>(out + (size_t)row * PCAP + cg * 16);
    dst[0] = make_uint4(c[q][0], c[q][1], c[q][2], c[q][3]);
    dst[1] = make_uint4(c[q][4], c[q][5], c[q][6], c[q][7]);
    if (row < r) {
#pragma unroll
      for (int p = 0; p < 8; ++p)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int cc = cg * 16 + 2 * p + h;
          const int x = (c[q][p] >> (16 * h)) & 0xFFFF;
          if (cc < r) {
            mx = max(mx, x);
            if (x >= (int)PC16) over = 1;
          }
        }
    }
  }
  __syncthreads();
  if (mx) atomicMax(&s_max, mx);
  if (over) s_over = 1;
  __syncthreads();
  if (tid == 0) {
    atomicMax(stats + 0, s_max);
    if (s_over) atomicOr(stats + 1, 1);
  }
}

__global__ void k_bnd_fill(int32_t *dB, int32_t Np) {
  const int64_t tot = (int64_t)Np * Np;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x)
    dB[e] = (e / Np == e % Np) ? 0 : INF;
}

// the cliques d_i(b, b') of (3), one CTA per region
__global__ void k_bnd_clique(const uint16_t *__restrict__ LR, const int32_t *__restrict__ bcnt,
                             const int32_t *__restrict__ boff, int32_t *dB, int32_t ldB) {
  const int i = blockIdx.x;
  const int nb = bcnt[i], b0 = boff[i];
  const uint16_t *L = LR + (size_t)i * PCAP * PCAP;
  for (int e = threadIdx.x; e < nb * nb; e += blockDim.x) {
    const int a = e / nb, b = e % nb;
    const uint32_t x = L[a * PCAP + b];
    dB[(int64_t)(b0 + a) * ldB + b0 + b] = x >= PC16 ? INF : (int32_t)x;
  }
}

// the arcs of G^r that join two regions (both ends are boundary vertices)
__global__ void k_bnd_cross(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                            const int32_t *__restrict__ w, const int32_t *__restrict__ bvert, int32_t NB,
                            const int32_t *__restrict__ reg, const int32_t *__restrict__ gidx, int32_t *dB,
                            int32_t ldB) {
  for (int32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < NB; g += gridDim.x * blockDim.x) {
    const int32_t v = bvert[g], rv = reg[v];
    for (int32_t a = rowptr[v], e = rowptr[v + 1]; a < e; ++a) {
      const int32_t x = col[a];
      if (reg[x] != rv) atomicMin(&dB[(int64_t)g * ldB + gidx[x]], w[a]);
    }
  }
}

__global__ void k_bnd_lab(const int32_t *__restrict__ bvert, const int32_t *__restrict__ cc, int32_t NB, int32_t Np,
                          int32_t *labB) {
  for (int32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < Np; g += gridDim.x * blockDim.x)
    labB[g] = g < NB ? cc[bvert[g]] : -1 - g;
}

// u16 copy of the boundary distances (0xFFFF = INF or >= 0xFFFF), and the largest finite one
__global__ void k_bnd_narrow(const int32_t *__restrict__ dB, int32_t ldB, int32_t NB, int32_t NBp, uint16_t *dB16,
                             int32_t *stats) {
  const int64_t tot = (int64_t)NB * (NBp / 2);
  int mx = 0;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t g = (int32_t)(e / (NBp / 2)), h = (int32_t)(e % (NBp / 2)) * 2;
    uint32_t pr = 0;
#pragma unroll
    for (int t = 0; t < 2; ++t) {
      uint32_t x = 0xFFFFu;
      if (h + t < NB) {
        const int32_t d = dB[(int64_t)g * ldB + h + t];
        if (d < INF) mx = max(mx, d);
        x = d < 0xFFFF ? (uint32_t)d : 0xFFFFu;
      }
      pr |= x << (16 * t);
    }
    reinterpret_cast<uint32_t *>(dB16 + (int64_t)g * NBp)[h / 2] = pr;
  }
  for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(stats, mx);
}

// Min-plus product of region i (blockIdx.y) with its boundary as the inner dimension, one 128-column
// block (blockIdx.x) per CTA; thread (rg, cg) owns rows rg*8..+8 and columns cg*16..+16 (8 x 8 pairs).
//   FINAL = false, (2):  DBVt[v][g] = min_{b < |B_i|} d_i(v, b) + dB16[boff_i + b][g]     (v in R_i)
//   FINAL = true,  (1):  D16[u][v]  = min( [v in R_i] d_i(u, v), min_b d_i(u, b) + DBVt[v][boff_i + b] ),
//                        INF when u and v lie in different components (then sums may have wrapped)
// A = d_i(., B_i) staged per 32-deep chunk as duplicated u32 (row b of the symmetric d_i, coalesced);
// chunk tails padded with the neutral pair (A = 0xFFFF, B = 0: the sum is 0xFFFF and never wins).
template <bool FINAL>
__global__ void __launch_bounds__(MP_NT)
    k_region_mp(const uint16_t *__restrict__ LR, const int32_t *__restrict__ roff, const int32_t *__restrict__ bcnt,
                const int32_t *__restrict__ boff, const int32_t *__restrict__ perm, const uint16_t *__restrict__ Bsrc,
                int64_t ldb, int32_t ncols, uint16_t *__restrict__ out, int64_t ldo, const int32_t *__restrict__ reg,
                const int32_t *__restrict__ loc, const int32_t *__restrict__ cc, const int32_t *__restrict__ rcomp,
                int32_t multi, const int32_t *__restrict__ rlist, const int32_t *__restrict__ stats,
                const int32_t *__restrict__ rneed) {
  __shared__ __align__(16) uint32_t As[MP_KC][PCAP];
  if (stats[1] || stats[0] + stats[2] >= 0xFFFF || (FINAL && stats[0] + stats[3] >= 0xFFFF)) return;
  if (rneed && !rneed[rlist ? rlist[blockIdx.y] : blockIdx.y]) return;
  __shared__ __align__(16) uint16_t Bs[MP_KC][MP_BS];
  __shared__ int32_t cl[MP_TC], ccol[MP_TC];
  const int i = rlist ? rlist[blockIdx.y] : blockIdx.y, tid = threadIdx.x;
  const int32_t r0 = roff[i], r = roff[i + 1] - r0, nb = bcnt[i], b0 = boff[i];
  const int32_t c0 = blockIdx.x * MP_TC;
  const uint16_t *L = LR + (size_t)i * PCAP * PCAP;
  const int rg = tid >> 3, cg = tid & 7;
  if (FINAL && tid < MP_TC) {
    const int32_t v = c0 + tid;
    int32_t lc = -1, cv = 0;
    if (v < ncols) {
      if (reg[v] == i) lc = loc[v];
      if (multi) cv = cc[v];
    }
    cl[tid] = lc;
    ccol[tid] = cv;
  }
  uint32_t acc[8][8];
#pragma unroll
  for (int q = 0; q < 8; ++q)
#pragma unroll
    for (int p = 0; p < 8; ++p) acc[q][p] = 0xFFFFFFFFu;
  const bool active = rg * 8 < r;
  for (int kb = 0; kb < nb; kb += MP_KC) {
    const int kc = min(MP_KC, nb - kb), kc8 = (kc + 7) & ~7;
    __syncthreads();
    for (int e = tid; e < kc8 * PCAP; e += MP_NT) {
      const int k = e / PCAP, u = e % PCAP;
      As[k][u] = (k < kc && u < r) ? dup16(L[(kb + k) * PCAP + u]) : 0xFFFFFFFFu;
    }
    if (!FINAL) {
      for (int e = tid; e < kc8 * (MP_TC / 8); e += MP_NT) {
        const int k = e / (MP_TC / 8), c8 = (e % (MP_TC / 8)) * 8;
        uint4 x = make_uint4(0, 0, 0, 0);
        if (k < kc) x = *reinterpret_cast<const uint4 *>(Bsrc + (int64_t)(b0 + kb + k) * ldb + c0 + c8);
        *reinterpret_cast<uint4 *>(&Bs[k][c8]) = x;
      }
    } else {
      for (int e = tid; e < kc8 * MP_TC; e += MP_NT) {
        const int c = e / kc8, k = e % kc8;
        uint16_t x = 0;
        if (k < kc) x = c0 + c < ncols ? Bsrc[(int64_t)(c0 + c) * ldb + b0 + kb + k] : (uint16_t)0xFFFF;
        Bs[k][c] = x;
      }
    }
    __syncthreads();
    if (active) {
      for (int k = 0; k < kc8; ++k) {
        const uint4 a0 = *reinterpret_cast<const uint4 *>(&As[k][rg * 8]);
        const uint4 a1 = *reinterpret_cast<const uint4 *>(&As[k][rg * 8 + 4]);
        const uint4 x0 = *reinterpret_cast<const uint4 *>(&Bs[k][cg * 16]);
        const uint4 x1 = *reinterpret_cast<const uint4 *>(&Bs[k][cg * 16 + 8]);
        const uint32_t a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const uint32_t b[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
#pragma unroll
        for (int q = 0; q < 8; ++q)
#pragma unroll
          for (int p = 0; p < 8; ++p) acc[q][p] = __viaddmin_u16x2(a[q], b[p], acc[q][p]);
      }
    }
  }
  if (FINAL) __syncthreads();   // cl / ccol visible (nb == 0: no barrier in the loop)
  if (!active) return;
  const int32_t rc = multi ? rcomp[i] : 0;
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const int u = rg * 8 + q;
    if (u >= r) break;
    const int32_t vu = perm[r0 + u];
    uint32_t o[8];
#pragma unroll
    for (int p = 0; p < 8; ++p) o[p] = acc[q][p];
    if (FINAL) {
#pragma unroll
      for (int p = 0; p < 8; ++p) {
        uint32_t lo = o[p] & 0xFFFFu, hi = o[p] >> 16;
        const int ca = cg * 16 + 2 * p;
        if (cl[ca] >= 0) lo = min(lo, (uint32_t)L[u * PCAP + cl[ca]]);
        if (cl[ca + 1] >= 0) hi = min(hi, (uint32_t)L[u * PCAP + cl[ca + 1]]);
        if (c0 + ca >= ncols || (multi && ccol[ca] != rc)) lo = 0xFFFFu;
        if (c0 + ca + 1 >= ncols || (multi && ccol[ca + 1] != rc)) hi = 0xFFFFu;
        o[p] = lo | (hi << 16);
      }
    }
    uint16_t *dst = out + (int64_t)vu * ldo + c0 + cg * 16;
    if (c0 + cg * 16 < ldo) *reinterpret_cast<uint4 *>(dst) = make_uint4(o[0], o[1], o[2], o[3]);
    if (c0 + cg * 16 + 8 < ldo) *reinterpret_cast<uint4 *>(dst + 8) = make_uint4(o[4], o[5], o[6], o[7]);
  }
}

// DBV[g][v] = DBVt[v][g]: the boundary rows of d as the final product stages them (rows contiguous in v)
constexpr int TR = 64;
__global__ void k_transpose16(const uint16_t *__restrict__ in, int64_t ldi, int32_t rows, int32_t cols,
                              uint16_t *__restrict__ out, int64_t ldo, int32_t *mx_out) {
  __shared__ uint16_t tile[TR][TR + 2];
  const int r0 = blockIdx.y * TR, c0 = blockIdx.x * TR;
  uint32_t mx = 0;   // largest entry < 0xFFFF (the no-wrap guard of product (1))
  for (int e = threadIdx.x; e < TR * TR; e += blockDim.x) {
    const int r = e / TR, c = e % TR;
    if (r0 + r < rows && c0 + c < cols) {
      const uint16_t x = in[(int64_t)(r0 + r) * ldi + c0 + c];
      tile[r][c] = x;
      if (x != 0xFFFF) mx = max(mx, (uint32_t)x);
    }
  }
  __syncthreads();
  for (int e = threadIdx.x; e < TR * TR; e += blockDim.x) {
    const int c = e / TR, r = e % TR;
    if (r0 + r < rows && c0 + c < cols) out[(int64_t)(c0 + c) * ldo + r0 + r] = tile[r][c];
  }
  for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(mx_out, (int32_t)mx);
}

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem, int bytes) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(bytes));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;\n" ::: "memory"); }

// The two products for the regions with |B_i| <= MP_KC, persistent.
//   FINAL = false, (2): DBVt[v][g] = min_b d_i(v, b) + dB16[boff_i + b][g]   (B rows: dB16, row-major in g)
//   FINAL = true,  (1): D16[u][v]  = min([v in R_i] d_i(u, v), min_b d_i(u, b) + DBV[boff_i + b][v]), INF
//                       across components
// The tile of region i is its r_i rows x W_i columns, W_i = 16 * min(32, 256 / ceil(r_i / 8)) (every
// thread busy whatever the region size: thread (ro, cg) owns rows ro*8..+8 and columns cg*16..+16); a CTA
// walks a contiguous range of (region, tile) items in region-major order, so A = d_i(., B_i) is staged
// once per region, and the B rows of the next tile stream into the other half of a double buffer by
// cp.async while the current tile is computed.  Only tiles that meet the region's vertex-id range look
// for local columns.  Guard (uniform): nothing runs unless the u16 sums of this product cannot wrap,
// stats[0] (Lmax) + stats[2] (max of dB) < 0xFFFF, for FINAL also stats[0] + stats[3] (max of DBV) <
// 0xFFFF, and no region overflowed.
constexpr int FW_MAXW = 128, FW_BS = FW_MAXW + 8;
__device__ __forceinline__ int width_of(int32_t r) { return 16 * min(FW_MAXW / 16, PR_NT / max(1, (r + 7) >> 3)); }

template <bool FINAL>
__global__ void __launch_bounds__(PR_NT, PR_MIN)
    k_region_prod(const uint16_t *__restrict__ LR, const int32_t *__restrict__ roff, const int32_t *__restrict__ bcnt,
                  const int32_t *__restrict__ boff, const int32_t *__restrict__ perm,
                  const uint16_t *__restrict__ Bsrc, int64_t ldb, int32_t ncols, uint16_t *__restrict__ out,
                  int64_t ldo, const int32_t *__restrict__ reg, const int32_t *__restrict__ loc,
                  const int32_t *__restrict__ cc, const int32_t *__restrict__ rcomp, const int2 *__restrict__ vrange,
                  int32_t multi, const int32_t *__restrict__ itemoff, int32_t K, const int32_t *__restrict__ stats) {
  extern __shared__ __align__(16) uint8_t smraw[];
  uint32_t(*As)[PCAP] = reinterpret_cast<uint32_t(*)[PCAP]>(smraw);                                // [MP_KC][PCAP]
  uint16_t(*Bs)[MP_KC][FW_BS] = reinterpret_cast<uint16_t(*)[MP_KC][FW_BS]>(smraw + MP_KC * PCAP * 4);  // [2]
  __shared__ int32_t cl[FINAL ? FW_MAXW : 1], ccol[FINAL ? FW_MAXW : 1];
  if (stats[1] || stats[0] + stats[2] >= 0xFFFF || (FINAL && stats[0] + stats[3] >= 0xFFFF)) return;
  const int tid = threadIdx.x;
  const int32_t total = itemoff[K];
  const int32_t t0 = (int32_t)((int64_t)total * blockIdx.x / gridDim.x);
  const int32_t t1 = (int32_t)((int64_t)total * (blockIdx.x + 1) / gridDim.x);
  if (t0 >= t1) return;
  // region of item t: itemoff is monotone, items are visited in order
  int ri = 0;
  {
    int lo = 0, hi = K - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (itemoff[mid] <= t0) lo = mid; else hi = mid - 1;
    }
    ri = lo;
  }
  // the next tile's B rows: region i, tile t (every thread issues its share of the 16-byte chunks)
  auto issue = [&](int32_t t, int i, int32_t nb, int32_t b0, int32_t W, int buf) {
    const int32_t c0 = (t - itemoff[i]) * W;
    const int chunks = W / 8;
    for (int e = tid; e < nb * chunks; e += PR_NT) {
      const int k = e / chunks, c8 = (e % chunks) * 8;
      const bool ok = c0 + c8 < ldb;
      cp_async16(&Bs[buf][k][c8], Bsrc + (int64_t)(b0 + k) * ldb + (ok ? c0 + c8 : 0), ok ? 16 : 0);
    }
    cp_async_commit();
  };
  __shared__ int32_t s_perm[PCAP];
  int cur = -1, buf = 0;
  int32_t r0 = 0, r = 0, nb = 0, b0 = 0, W = 16, cgs = 1, nro = 0, cgi = 0, ro = 0, i_off = 0;
  int32_t i_end = itemoff[ri + 1];   // first item past region ri (kept in a register)
  int2 vr = make_int2(0, -1);
  {
    const int32_t rr = roff[ri + 1] - roff[ri];
    issue(t0, ri, bcnt[ri], boff[ri], width_of(rr), 0);
  }
  for (int32_t t = t0; t < t1; ++t) {
    while (i_end <= t) i_end = itemoff[++ri + 1];
    const int i = ri;
    __syncthreads();   // tile t-1 is done with As, Bs[buf ^ 1], cl, s_perm
    if (i != cur) {    // per-region constants and staging: A, the member ids
      cur = i;
      r0 = roff[i], r = roff[i + 1] - r0, nb = bcnt[i], b0 = boff[i];
      nro = (r + 7) >> 3, W = width_of(r), cgs = W / 16, cgi = tid % cgs, ro = tid / cgs;
      i_off = itemoff[i];
      if (FINAL) vr = vrange[i];
      const uint16_t *L = LR + (size_t)i * PCAP * PCAP;
      for (int e = tid; e < nb * PCAP; e += PR_NT) {
        const int k = e / PCAP, u = e % PCAP;
        As[k][u] = u < r ? dup16(L[k * PCAP + u]) : 0xFFFFFFFFu;
      }
      for (int u = tid; u < r; u += PR_NT) s_perm[u] = perm[r0 + u];
    }
    const int32_t c0 = (t - i_off) * W;
    int loc_any = 0;
    if (FINAL) {
      const bool meets = c0 <= vr.y && c0 + W > vr.x;
      if (meets || multi) {
        for (int c = tid; c < W; c += PR_NT) {
          const int32_t v = c0 + c;
          int32_t lc = -1, cv = 0;
          if (v < ncols) {
            if (meets && reg[v] == i) lc = loc[v];
            if (multi) cv = cc[v];
          }
          cl[c] = lc;
          ccol[c] = cv;
          loc_any |= lc >= 0;
        }
      }
    }
    if (t + 1 < t1) {
      if (i_end > t + 1) {
        issue(t + 1, i, nb, b0, W, buf ^ 1);
      } else {
        int in = i + 1;
        while (itemoff[in + 1] <= t + 1) ++in;
        issue(t + 1, in, bcnt[in], boff[in], width_of(roff[in + 1] - roff[in]), buf ^ 1);
      }
    } else {
      cp_async_commit();   // keep the group count uniform
    }
    cp_async_wait1();
    loc_any = __syncthreads_or(loc_any);
    if (ro < nro) {
      uint32_t acc[8][8];
#pragma unroll
      for (int q = 0; q < 8; ++q)
#pragma unroll
        for (int p = 0; p < 8; ++p) acc[q][p] = 0xFFFFFFFFu;
      const uint16_t *bsrc = &Bs[buf][0][cgi * 16];
      for (int k = 0; k < nb; ++k) {
        const uint4 a0 = *reinterpret_cast<const uint4 *>(&As[k][ro * 8]);
        const uint4 a1 = *reinterpret_cast<const uint4 *>(&As[k][ro * 8 + 4]);
        const uint4 x0 = *reinterpret_cast<const uint4 *>(bsrc + k * FW_BS);
        const uint4 x1 = *reinterpret_cast<const uint4 *>(bsrc + k * FW_BS + 8);
        const uint32_t a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const uint32_t b[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
#pragma unroll
        for (int q = 0; q < 8; ++q)
#pragma unroll
          for (int p = 0; p < 8; ++p) acc[q][p] = __viaddmin_u16x2(a[q], b[p], acc[q][p]);
      }
      const uint16_t *L = LR + (size_t)i * PCAP * PCAP;
      const int rc = FINAL && multi ? rcomp[i] : 0;
      const bool fix = FINAL && (loc_any || multi || c0 + W > ncols);
      const int cb = c0 + cgi * 16;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const int u = ro * 8 + q;
        if (u < r) {
          uint32_t o[8];
#pragma unroll
          for (int p = 0; p < 8; ++p) o[p] = acc[q][p];
          if (fix) {
#pragma unroll
            for (int p = 0; p < 8; ++p) {
              uint32_t lo = o[p] & 0xFFFFu, hi = o[p] >> 16;
              const int ca = cgi * 16 + 2 * p;
              if (loc_any) {
                if (cl[ca] >= 0) lo = min(lo, (uint32_t)L[u * PCAP + cl[ca]]);
                if (cl[ca + 1] >= 0) hi = min(hi, (uint32_t)L[u * PCAP + cl[ca + 1]]);
              }
              if (c0 + ca >= ncols || (multi && ccol[ca] != rc)) lo = 0xFFFFu;
              if (c0 + ca + 1 >= ncols || (multi && ccol[ca + 1] != rc)) hi = 0xFFFFu;
              o[p] = lo | (hi << 16);
            }
          }
          uint16_t *dst = out + (int64_t)s_perm[u] * ldo + cb;
          if (cb < ldo) *reinterpret_cast<uint4 *>(dst) = make_uint4(o[0], o[1], o[2], o[3]);
          if (cb + 8 < ldo) *reinterpret_cast<uint4 *>(dst + 8) = make_uint4(o[4], o[5], o[6], o[7]);
        }
      }
    }
    buf ^= 1;
  }
}

constexpr int FINAL_SMEM = MP_KC * PCAP * 4 + 2 * MP_KC * FW_BS * 2;

// item offsets of k_region_prod: region i contributes ceil(ncols / W_i) tiles (none when |B_i| > MP_KC:
// the general kernel does it); one CTA, chunked block scan
__global__ void __launch_bounds__(1024) k_items(const int32_t *__restrict__ roff, const int32_t *__restrict__ bcnt,
                                                int32_t K, int32_t ncols, const int32_t *__restrict__ rneed,
                                                int32_t *itemoff) {
  __shared__ int32_t part[1024];
  __shared__ int32_t carry;
  if (threadIdx.x == 0) carry = 0;
  for (int base = 0; base < K; base += 1024) {
    const int i = base + threadIdx.x;
    int32_t c = 0;
    if (i < K && bcnt[i] <= MP_KC && (!rneed || rneed[i]))
      c = (ncols + width_of(roff[i + 1] - roff[i]) - 1) / width_of(roff[i + 1] - roff[i]);
    part[threadIdx.x] = c;
    __syncthreads();
    for (int o = 1; o < 1024; o <<= 1) {   // inclusive Hillis-Steele scan
      const int32_t x = threadIdx.x >= o ? part[threadIdx.x - o] : 0;
      __syncthreads();
      part[threadIdx.x] += x;
      __syncthreads();
    }
    if (i < K) itemoff[i + 1] = carry + part[threadIdx.x];
    __syncthreads();
    if (threadIdx.x == 1023) carry += part[1023];
    __syncthreads();
  }
  if (threadIdx.x == 0) itemoff[0] = 0;
}

// The boundary graph H of a level: vertex g = global boundary index; arcs: the clique of its region's
// boundary with weights d_i (local indices: the boundary comes first in a region) and its joining arcs.
__global__ void k_h_deg(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                        const int32_t *__restrict__ bvert, int32_t NB, const int32_t *__restrict__ reg,
                        const int32_t *__restrict__ bcnt, int32_t *deg) {
  for (int32_t g = blockIdx.x * blockDim.x + threadIdx.x; g <= NB; g += gridDim.x * blockDim.x) {
    if (g == NB) {
      deg[g] = 0;
      continue;
    }
    const int32_t v = bvert[g], i = reg[v];
    int32_t d = bcnt[i] - 1;
    for (int32_t a = rowptr[v], e = rowptr[v + 1]; a < e; ++a) d += reg[col[a]] != i;
    deg[g] = d;
  }
}

__global__ void k_h_fill(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                         const int32_t *__restrict__ w, const int32_t *__restrict__ bvert, int32_t NB,
                         const int32_t *__restrict__ reg, const int32_t *__restrict__ gidx,
                         const int32_t *__restrict__ bcnt, const int32_t *__restrict__ boff,
                         const uint16_t *__restrict__ LR, const int32_t *__restrict__ hrow, int32_t *hcol, int32_t *hw) {
  for (int32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < NB; g += gridDim.x * blockDim.x) {
    const int32_t v = bvert[g], i = reg[v], b0 = boff[i], nb = bcnt[i], a = g - b0;
    const uint16_t *L = LR + (size_t)i * PCAP * PCAP + (size_t)a * PCAP;
    int32_t pos = hrow[g];
    for (int32_t b = 0; b < nb; ++b) {
      if (b == a) continue;
      hcol[pos] = b0 + b;
      hw[pos] = L[b];
      ++pos;
    }
    for (int32_t t = rowptr[v], e = rowptr[v + 1]; t < e; ++t) {
      const int32_t x = col[t];
      if (reg[x] == i) continue;
      hcol[pos] = gidx[x];
      hw[pos] = w[t];
      ++pos;
    }
  }
}

// components of H are those of the graph restricted to its boundary (a component with two or more regions
// has all its boundary vertices connected through the cliques and joining arcs); label = smallest g.
// Two passes: hcc == nullptr -> mn[cc] = min g; else hcc[g] = mn[cc(g)]
__global__ void k_h_cc(const int32_t *__restrict__ bvert, const int32_t *__restrict__ cc, int32_t NB, int32_t *mn,
                       int32_t *hcc) {
  for (int32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < NB; g += gridDim.x * blockDim.x) {
    const int32_t c = cc[bvert[g]];
    if (hcc) hcc[g] = mn[c];
    else atomicMin(&mn[c], g);
  }
}

// largest entry < 0xFFFF of the first `cols` columns of a u16 matrix (rows x ld, ld % 8 == 0)
__global__ void k_max16(const uint16_t *__restrict__ M, int32_t rows, int64_t ld, int32_t cols, int32_t *out) {
  const int64_t tot = (int64_t)rows * (ld / 8);
  uint32_t mx = 0;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c8 = (int32_t)(e % (ld / 8)) * 8;
    if (c8 >= cols) continue;
    const uint4 v = reinterpret_cast<const uint4 *>(M)[e];
    const uint32_t w4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const uint32_t lo = w4[j] & 0xFFFFu, hi = w4[j] >> 16;
      if (lo != 0xFFFFu && c8 + 2 * j < cols) mx = max(mx, lo);
      if (hi != 0xFFFFu && c8 + 2 * j + 1 < cols) mx = max(mx, hi);
    }
  }
  for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(out, (int32_t)mx);
}

// All of the region labelling in one cooperative launch (grid-wide barriers between BFS levels): seeds,
// Jacobi BFS levels until nothing changes, then -- while a cell exceeds PCAP -- counts, the denser
// seeds of the oversized cells and BFS again inside them.  The final labels end in lab0.
// st[0]: an unlabelled vertex remained; st[1]: passes; st[2]: did not converge; st[4..6]: level flags
__global__ void __launch_bounds__(NT) k_partition(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                  const int32_t *__restrict__ cc, int32_t n, int32_t S, int32_t *lab0,
                                                  int32_t *lab1, int32_t *grp, int32_t *cnt, int32_t *st) {
  namespace cg = cooperative_groups;
  cg::grid_group grid = cg::this_grid();
  const int32_t tid0 = blockIdx.x * blockDim.x + threadIdx.x, stride = gridDim.x * blockDim.x;
  for (int32_t v = tid0; v < n; v += stride) {
    lab0[v] = (v % S == 0 || cc[v] == v) ? v : -1;
    grp[v] = 0;
  }
  if (tid0 == 0) st[4] = st[5] = st[6] = 0;
  grid.sync();
  int32_t *lin = lab0, *lout = lab1;
  int32_t S2 = max(1, S / 2);
  int level = 0;
  for (int pass = 1;; ++pass) {
    for (;; ++level) {
      const int f = level % 3;
      int ch = 0;
      for (int32_t v = tid0; v < n; v += stride) {
        int32_t l = lin[v];
        if (l < 0) {
          const int32_t g = grp[v];
          int32_t m = INT_MAX;
          for (int32_t a = rowptr[v], e = rowptr[v + 1]; a < e; ++a) {
            const int32_t u = col[a];
            const int32_t lu = lin[u];
            if (lu >= 0 && grp[u] == g) m = min(m, lu);
          }
          if (m != INT_MAX) {
            l = m;
            ch = 1;
          }
        }
        lout[v] = l;
      }
      if (__syncthreads_or(ch) && threadIdx.x == 0) st[4 + f] = 1;
      if (tid0 == 0) st[4 + (level + 1) % 3] = 0;   // read two levels ago, before the last barrier
      grid.sync();
      int32_t *x = lin;
      lin = lout;
      lout = x;
      if (!st[4 + f]) break;
      if (level > 4 * n + 8) {
        if (tid0 == 0) st[2] = 1;
        break;
      }
    }
    ++level;   // the flag of the level that ended the BFS is not reused before it is cleared
    // cell sizes, then the oversized cells get denser seeds (grp = old cell: the next BFS stays inside)
    for (int32_t v = tid0; v < n; v += stride) cnt[v] = 0;
    if (tid0 == 0) st[7] = 0;
    grid.sync();
    for (int32_t v = tid0; v < n; v += stride) {
      const int32_t l = lin[v];
      if (l < 0) st[0] = 1;
      else atomicAdd(&cnt[l], 1);
    }
    grid.sync();
    int o = 0;
    for (int32_t v = tid0; v < n; v += stride) {
      const int32_t l = lin[v];
      grp[v] = l;
      if (l >= 0 && cnt[l] > PCAP) {
        lin[v] = (v == l || v % S2 == 0) ? v : -1;
        o = 1;
      }
    }
    if (__syncthreads_or(o) && threadIdx.x == 0) st[7] = 1;
    grid.sync();
    if (!st[7] || st[2] || pass > 12) {
      if (tid0 == 0) st[1] = pass;
      if (lin != lab0)
        for (int32_t v = tid0; v < n; v += stride) lab0[v] = lin[v];
      if (pass > 12 && st[7] && tid0 == 0) st[2] = 1;
      return;
    }
    S2 = max(1, S2 / 2);
  }
}

// per-region statistics and lists on the device (K = tot[0]): max |B_i|, sum |R_i||B_i|, several
// components, the regions with |B_i| > MP_KC, the vertex-id range of every region
__global__ void k_region_stats(const int32_t *__restrict__ perm, const int32_t *__restrict__ roff,
                               const int32_t *__restrict__ bcnt, const int32_t *__restrict__ rcomp, int32_t *tot,
                               int32_t *big, int2 *vr) {
  const int32_t K = tot[0];
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < K; i += gridDim.x * blockDim.x) {
    const int32_t b = bcnt[i], r = roff[i + 1] - roff[i];
    atomicMax(&tot[3], b);
    atomicAdd(reinterpret_cast<unsigned long long *>(tot + 6), (unsigned long long)r * b);
    if (rcomp[i] != rcomp[0]) tot[4] = 1;
    if (b > MP_KC) big[atomicAdd(&tot[5], 1)] = i;
    int32_t lo = INT_MAX, hi = -1;
    for (int32_t e = roff[i]; e < roff[i + 1]; ++e) {
      lo = min(lo, perm[e]);
      hi = max(hi, perm[e]);
    }
    vr[i] = make_int2(lo, hi);
  }
}

// ----------------------------------------------------------------------------------------------
// Dense FW on a small boundary matrix (|B| up to a few thousand) with 64 x 64 tiles, packed u16x2 capped
// at PC16 (the argument of sec. 6a: exact below the cap), the whole schedule in one cooperative launch:
// per round k, block 0 closes the pivot tile (64 barriers in shared memory), every block then takes
// pivot-row tiles (k, j) -- written with their transposes (j, k), D stays symmetric -- and then upper
// tiles (i <= j) of the rest, each written with its mirror; grid barriers between the three phases.
// 128-row tiles (the TMA kernel of sec. 6a) leave this size latency bound: a round costs its serial
// 128-step phase 1 and two tile-deep launches (~85 us at |B| ~ 1,000).
constexpr int F64 = 64;
__device__ __forceinline__ void f64_load(uint16_t (*dst)[F64], const uint16_t *M, int64_t ld, int ti, int tj) {
  for (int e = threadIdx.x; e < F64 * F64 / 8; e += blockDim.x) {
    const int r = e / 8, c8 = (e % 8) * 8;
    *reinterpret_cast<uint4 *>(&dst[r][c8]) =
        *reinterpret_cast<const uint4 *>(M + (int64_t)(ti * F64 + r) * ld + tj * F64 + c8);
  }
}
// C (4 rows x 4 columns per thread) = min(C, A^T (x) B): A[m][r] (row m of the pivot-row tile of i), B[m][c]
__device__ __forceinline__ void f64_mp(const uint16_t (*A)[F64], const uint16_t (*B)[F64], uint32_t c[4][2]) {
  const int tr = threadIdx.x / 16, tc = threadIdx.x % 16;
#pragma unroll 8
  for (int m = 0; m < F64; ++m) {
    const uint2 av = *reinterpret_cast<const uint2 *>(&A[m][tr * 4]);
    const uint2 bv = *reinterpret_cast<const uint2 *>(&B[m][tc * 4]);
    const uint32_t a[4] = {dup16(av.x & 0xFFFFu), dup16(av.x >> 16), dup16(av.y & 0xFFFFu), dup16(av.y >> 16)};
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      c[q][0] = __viaddmin_u16x2(a[q], bv.x, c[q][0]);
      c[q][1] = __viaddmin_u16x2(a[q], bv.y, c[q][1]);
    }
  }
}
// write the thread's 4 x 4 block into tile (ti, tj) and -- mirror -- its transpose into (tj, ti)
__device__ __forceinline__ void f64_store(uint16_t *M, int64_t ld, int ti, int tj, const uint32_t c[4][2], bool mirror) {
  const int tr = threadIdx.x / 16, tc = threadIdx.x % 16;
#pragma unroll
  for (int q = 0; q < 4; ++q)
    *reinterpret_cast<uint2 *>(M + (int64_t)(ti * F64 + tr * 4 + q) * ld + tj * F64 + tc * 4) = make_uint2(c[q][0], c[q][1]);
  if (mirror) {
#pragma unroll
    for (int cc = 0; cc < 4; ++cc) {   // column tc*4+cc of the block = row of the transpose
      const uint32_t lo = (c[0][cc >> 1] >> (16 * (cc & 1))) & 0xFFFFu, l1 = (c[1][cc >> 1] >> (16 * (cc & 1))) & 0xFFFFu;
      const uint32_t l2 = (c[2][cc >> 1] >> (16 * (cc & 1))) & 0xFFFFu, l3 = (c[3][cc >> 1] >> (16 * (cc & 1))) & 0xFFFFu;
      *reinterpret_cast<uint2 *>(M + (int64_t)(tj * F64 + tc * 4 + cc) * ld + ti * F64 + tr * 4) =
          make_uint2(lo | (l1 << 16), l2 | (l3 << 16));
    }
  }
}
__global__ void __launch_bounds__(256) k_fw64(uint16_t *M, int32_t N) {
  namespace cg = cooperative_groups;
  cg::grid_group grid = cg::this_grid();
  __shared__ __align__(16) uint16_t As[F64][F64], Bs[F64][F64];
  const int T = N / F64, tid = threadIdx.x, tr = tid / 16, tc = tid % 16;
  // phase 1 by block 0 (in shared memory, one barrier per step: an in-place step kk only reads row and
  // column kk, which it does not change)
  auto close_pivot = [&](int k) {
    f64_load(As, M, N, k, k);
    __syncthreads();
    for (int kk = 0; kk < F64; ++kk) {
      const uint2 bv = *reinterpret_cast<const uint2 *>(&As[kk][tc * 4]);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint32_t a = dup16(As[tr * 4 + q][kk]);
        uint2 cv = *reinterpret_cast<const uint2 *>(&As[tr * 4 + q][tc * 4]);
        cv.x = __viaddmin_u16x2(a, bv.x, cv.x);
        cv.y = __viaddmin_u16x2(a, bv.y, cv.y);
        *reinterpret_cast<uint2 *>(&As[tr * 4 + q][tc * 4]) = cv;
      }
      __syncthreads();
    }
  };
  auto store_tile = [&](int ti) {   // As -> tile (ti, ti)
#pragma unroll
    for (int q = 0; q < 4; ++q)
      *reinterpret_cast<uint2 *>(M + (int64_t)(ti * F64 + tr * 4 + q) * N + ti * F64 + tc * 4) =
          *reinterpret_cast<const uint2 *>(&As[tr * 4 + q][tc * 4]);
  };
  if (blockIdx.x == 0 && T > 0) {
    close_pivot(0);
    store_tile(0);
  }
  grid.sync();
  for (int k = 0; k < T; ++k) {
    // the closed pivot tile (stored before the last grid barrier by block 0)
    if (blockIdx.x < T - 1) {
      __syncthreads();
      f64_load(As, M, N, k, k);
      __syncthreads();
    }
    // phase 2: pivot-row tiles (k, j) = min(C, P (x) C); P is closed and symmetric, so A[m][r] = P[m][r]
    for (int jt = blockIdx.x; jt < T - 1; jt += gridDim.x) {
      const int j = jt < k ? jt : jt + 1;
      __syncthreads();
      f64_load(Bs, M, N, k, j);
      __syncthreads();
      uint32_t c[4][2];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint2 x = *reinterpret_cast<const uint2 *>(&Bs[tr * 4 + q][tc * 4]);
        c[q][0] = x.x, c[q][1] = x.y;
      }
      f64_mp(As, Bs, c);
      f64_store(M, N, k, j, c, true);
    }
    grid.sync();
    // phase 3: upper tiles (i <= j) off row / column k: C = min(C, row(k,i)^T (x) row(k,j)), mirrored.
    // Lookahead: block 0 first updates the NEXT pivot tile (k+1, k+1) and closes it (phase 1 of round
    // k+1) while the other blocks work through the rest of phase 3
    if (blockIdx.x == 0 && k + 1 < T) {
      __syncthreads();
      f64_load(Bs, M, N, k, k + 1);
      f64_load(As, M, N, k + 1, k + 1);
      __syncthreads();
      uint32_t c[4][2];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint2 x = *reinterpret_cast<const uint2 *>(&As[tr * 4 + q][tc * 4]);
        c[q][0] = x.x, c[q][1] = x.y;
      }
      f64_mp(Bs, Bs, c);
      __syncthreads();
#pragma unroll
      for (int q = 0; q < 4; ++q) *reinterpret_cast<uint2 *>(&As[tr * 4 + q][tc * 4]) = make_uint2(c[q][0], c[q][1]);
      __syncthreads();
      for (int kk = 0; kk < F64; ++kk) {   // close it in place (as close_pivot, from shared memory)
        const uint2 bv = *reinterpret_cast<const uint2 *>(&As[kk][tc * 4]);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint32_t a = dup16(As[tr * 4 + q][kk]);
          uint2 cv = *reinterpret_cast<const uint2 *>(&As[tr * 4 + q][tc * 4]);
          cv.x = __viaddmin_u16x2(a, bv.x, cv.x);
          cv.y = __viaddmin_u16x2(a, bv.y, cv.y);
          *reinterpret_cast<uint2 *>(&As[tr * 4 + q][tc * 4]) = cv;
        }
        __syncthreads();
      }
      store_tile(k + 1);
    }
    const int64_t nt = (int64_t)T * (T + 1) / 2;
    const int64_t skip = (int64_t)(k + 1) * (k + 2) / 2 + (k + 1);   // the tile (k+1, k+1): block 0 did it
    const int gb = gridDim.x > 1 ? (int)gridDim.x - 1 : 1;            // block 0 takes regular tiles only alone
    for (int64_t e = gridDim.x > 1 ? blockIdx.x - 1 : 0; e < nt && (gridDim.x == 1 || blockIdx.x > 0); e += gb) {
      if (k + 1 < T && e == skip) continue;
      int i = (int)((sqrt(8.0 * (double)e + 1.0) - 1.0) / 2.0);   // e -> (j = row of the triangle, i <= j)
      while ((int64_t)(i + 1) * (i + 2) / 2 <= e) ++i;
      while ((int64_t)i * (i + 1) / 2 > e) --i;
      const int jj = i, ii = (int)(e - (int64_t)i * (i + 1) / 2);
      if (ii == k || jj == k) continue;
      __syncthreads();
      f64_load(As, M, N, k, ii);
      f64_load(Bs, M, N, k, jj);
      __syncthreads();
      uint32_t c[4][2];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint2 x = *reinterpret_cast<const uint2 *>(M + (int64_t)(ii * F64 + tr * 4 + q) * N + jj * F64 + tc * 4);
        c[q][0] = x.x, c[q][1] = x.y;
      }
      f64_mp(As, Bs, c);
      f64_store(M, N, ii, jj, c, ii != jj);
    }
    grid.sync();
  }
}

// k_fw64 with split barriers (the default; EAR_FW64_SPLIT=0 runs k_fw64): block 0 does the pivot-row tile (k, k+1) itself,
// arrives at both barriers of round k at once and runs the update and closure of pivot k+1 while the other
// blocks finish round k; they wait for the published pivot (flag) instead of a grid barrier after it.
// Counters: bar[2k] (pivot row done), bar[2k+1] (round k done), bar[2T] = index of the last closed pivot + 1.
__device__ __forceinline__ int ld_acquire_gpu(const int *p) {
  int v;
  asm volatile("ld.acquire.gpu.global.s32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void sb_arrive(int *c) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(c, 1);
  }
}
__device__ __forceinline__ void sb_wait(const int *c, int target) {
  if (threadIdx.x == 0) {
    while (ld_acquire_gpu(c) < target) __nanosleep(64);
    __threadfence();
  }
  __syncthreads();
}
__device__ __forceinline__ void f64_close(uint16_t (*As)[F64]) {   // in place, one barrier per step
  const int tr = threadIdx.x / 16, tc = threadIdx.x % 16;
  for (int kk = 0; kk < F64; ++kk) {
    const uint2 bv = *reinterpret_cast<const uint2 *>(&As[kk][tc * 4]);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint32_t a = dup16(As[tr * 4 + q][kk]);
      uint2 cv = *reinterpret_cast<const uint2 *>(&As[tr * 4 + q][tc * 4]);
      cv.x = __viaddmin_u16x2(a, bv.x, cv.x);
      cv.y = __viaddmin_u16x2(a, bv.y, cv.y);
      *reinterpret_cast<uint2 *>(&As[tr * 4 + q][tc * 4]) = cv;
    }
    __syncthreads();
  }
}
__global__ void __launch_bounds__(256) k_fw64s(uint16_t *M, int32_t N, int *bar) {
  __shared__ __align__(16) uint16_t As[F64][F64], Bs[F64][F64];
  const int T = N / F64, tid = threadIdx.x, tr = tid / 16, tc = tid % 16;
  const int G = gridDim.x, b = blockIdx.x;   // G >= 2 (the host checks)
  int *piv = bar + 2 * T;
  auto tile_to_smem = [&](uint16_t (*S)[F64], const uint32_t c[4][2]) {
#pragma unroll
    for (int q = 0; q < 4; ++q) *reinterpret_cast<uint2 *>(&S[tr * 4 + q][tc * 4]) = make_uint2(c[q][0], c[q][1]);
  };
  auto store_diag = [&](int ti) {
#pragma unroll
    for (int q = 0; q < 4; ++q)
      *reinterpret_cast<uint2 *>(M + (int64_t)(ti * F64 + tr * 4 + q) * N + ti * F64 + tc * 4) =
          *reinterpret_cast<const uint2 *>(&As[tr * 4 + q][tc * 4]);
  };
  if (b == 0) {
    if (T > 0) {
      f64_load(As, M, N, 0, 0);
      __syncthreads();
      f64_close(As);
      store_diag(0);
    }
    __syncthreads();
    if (tid == 0) {
      __threadfence();
      atomicExch(piv, 1);
    }
    for (int k = 0; k < T; ++k) {
      if (k > 0) sb_wait(&bar[2 * (k - 1) + 1], G);   // round k-1 done everywhere
      if (k + 1 < T) {
        // As holds the closed pivot k; the pivot-row tile (k, k+1)
        __syncthreads();
        f64_load(Bs, M, N, k, k + 1);
        __syncthreads();
        uint32_t c[4][2];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint2 x = *reinterpret_cast<const uint2 *>(&Bs[tr * 4 + q][tc * 4]);
          c[q][0] = x.x, c[q][1] = x.y;
        }
        f64_mp(As, Bs, c);
        f64_store(M, N, k, k + 1, c, true);
        sb_arrive(&bar[2 * k]);
        sb_arrive(&bar[2 * k + 1]);
        // the next pivot: (k+1, k+1) = min(C, row(k,k+1)^T (x) row(k,k+1)), then closed
        tile_to_smem(Bs, c);
        f64_load(As, M, N, k + 1, k + 1);
        __syncthreads();
        uint32_t d[4][2];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint2 x = *reinterpret_cast<const uint2 *>(&As[tr * 4 + q][tc * 4]);
          d[q][0] = x.x, d[q][1] = x.y;
        }
        f64_mp(Bs, Bs, d);
        __syncthreads();
        tile_to_smem(As, d);
        __syncthreads();
        f64_close(As);
        store_diag(k + 1);
        __syncthreads();
        if (tid == 0) {
          __threadfence();
          atomicExch(piv, k + 2);
        }
      } else {
        sb_arrive(&bar[2 * k]);
        sb_arrive(&bar[2 * k + 1]);
      }
    }
    return;
  }
  const int gb = G - 1, bi = b - 1;
  for (int k = 0; k < T; ++k) {
    sb_wait(piv, k + 1);                              // pivot k closed
    if (k > 0) sb_wait(&bar[2 * (k - 1) + 1], G);     // round k-1 done everywhere
    // pivot-row tiles (k, j), j != k (and != k+1: block 0's)
    const int nrow = k + 1 < T ? T - 2 : T - 1;
    bool have_p = false;
    for (int jt = bi; jt < nrow; jt += gb) {
      int j = jt < k ? jt : jt + 1;   // skip k
      if (k + 1 < T && j >= k + 1) ++j;   // skip k+1
      __syncthreads();
      if (!have_p) {
        f64_load(As, M, N, k, k);
        have_p = true;
      }
      f64_load(Bs, M, N, k, j);
      __syncthreads();
      uint32_t c[4][2];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint2 x = *reinterpret_cast<const uint2 *>(&Bs[tr * 4 + q][tc * 4]);
        c[q][0] = x.x, c[q][1] = x.y;
      }
      f64_mp(As, Bs, c);
      f64_store(M, N, k, j, c, true);
    }
    sb_arrive(&bar[2 * k]);
    sb_wait(&bar[2 * k], G);
    const int64_t nt = (int64_t)T * (T + 1) / 2;
    const int64_t skip = (int64_t)(k + 1) * (k + 2) / 2 + (k + 1);   // (k+1, k+1): block 0's
    for (int64_t e = bi; e < nt; e += gb) {
      if (k + 1 < T && e == skip) continue;
      int i = (int)((sqrt(8.0 * (double)e + 1.0) - 1.0) / 2.0);
      while ((int64_t)(i + 1) * (i + 2) / 2 <= e) ++i;
      while ((int64_t)i * (i + 1) / 2 > e) --i;
      const int jj = i, ii = (int)(e - (int64_t)i * (i + 1) / 2);
      if (ii == k || jj == k) continue;
      __syncthreads();
      f64_load(As, M, N, k, ii);
      f64_load(Bs, M, N, k, jj);
      __syncthreads();
      uint32_t c[4][2];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint2 x = *reinterpret_cast<const uint2 *>(M + (int64_t)(ii * F64 + tr * 4 + q) * N + jj * F64 + tc * 4);
        c[q][0] = x.x, c[q][1] = x.y;
      }
      f64_mp(As, Bs, c);
      f64_store(M, N, ii, jj, c, ii != jj);
    }
    sb_arrive(&bar[2 * k + 1]);
  }
}

// The same 64-tile cooperative FW in int32 (one VIADDMNMX per min-plus, no cap): the boundary graphs
// whose distances pass the u16 kernel's 0x7FFF cap (cfg5's deeper levels) -- instead of the 128-tile
// TMA kernel, which is latency-bound at this size.  Thread (tr, tc) owns rows tr*4..+4, columns tc*4..+4.
__device__ __forceinline__ void f64i_load(int32_t (*dst)[F64], const int32_t *M, int64_t ld, int ti, int tj) {
  for (int e = threadIdx.x; e < F64 * F64 / 4; e += blockDim.x) {
    const int r = e / 16, c4 = (e % 16) * 4;
    *reinterpret_cast<int4 *>(&dst[r][c4]) = *reinterpret_cast<const int4 *>(M + (int64_t)(ti * F64 + r) * ld + tj * F64 + c4);
  }
}
__device__ __forceinline__ void f64i_mp(const int32_t (*A)[F64], const int32_t (*B)[F64], int32_t c[4][4]) {
  const int tr = threadIdx.x / 16, tc = threadIdx.x % 16;
#pragma unroll 8
  for (int m = 0; m < F64; ++m) {
    const int4 av = *reinterpret_cast<const int4 *>(&A[m][tr * 4]);
    const int4 bv = *reinterpret_cast<const int4 *>(&B[m][tc * 4]);
    const int32_t a[4] = {av.x, av.y, av.z, av.w}, b[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
    for (int q = 0; q < 4; ++q)
#pragma unroll
      for (int j = 0; j < 4; ++j) c[q][j] = __viaddmin_s32(a[q], b[j], c[q][j]);
  }
}
__device__ __forceinline__ void f64i_store(int32_t *M, int64_t ld, int ti, int tj, const int32_t c[4][4], bool mirror) {
  const int tr = threadIdx.x / 16, tc = threadIdx.x % 16;
#pragma unroll
  for (int q = 0; q < 4; ++q)
    *reinterpret_cast<int4 *>(M + (int64_t)(ti * F64 + tr * 4 + q) * ld + tj * F64 + tc * 4) =
        make_int4(c[q][0], c[q][1], c[q][2], c[q][3]);
  if (mirror)
#pragma unroll
    for (int j = 0; j < 4; ++j)
      *reinterpret_cast<int4 *>(M + (int64_t)(tj * F64 + tc * 4 + j) * ld + ti * F64 + tr * 4) =
          make_int4(c[0][j], c[1][j], c[2][j], c[3][j]);
}
__global__ void __launch_bounds__(256) k_fw64i(int32_t *M, int32_t N) {
  namespace cg = cooperative_groups;
  cg::grid_group grid = cg::this_grid();
  __shared__ __align__(16) int32_t As[F64][F64], Bs[F64][F64];
  const int T = N / F64, tid = threadIdx.x, tr = tid / 16, tc = tid % 16;
  auto close_tile = [&]() {   // As closed in place (an in-place step kk only reads row / column kk)
    for (int kk = 0; kk < F64; ++kk) {
      const int4 bv = *reinterpret_cast<const int4 *>(&As[kk][tc * 4]);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int32_t a = As[tr * 4 + q][kk];
        int4 cv = *reinterpret_cast<const int4 *>(&As[tr * 4 + q][tc * 4]);
        cv.x = __viaddmin_s32(a, bv.x, cv.x);
        cv.y = __viaddmin_s32(a, bv.y, cv.y);
        cv.z = __viaddmin_s32(a, bv.z, cv.z);
        cv.w = __viaddmin_s32(a, bv.w, cv.w);
        *reinterpret_cast<int4 *>(&As[tr * 4 + q][tc * 4]) = cv;
      }
      __syncthreads();
    }
  };
  auto store_tile = [&](int ti) {
#pragma unroll
    for (int q = 0; q < 4; ++q)
      *reinterpret_cast<int4 *>(M + (int64_t)(ti * F64 + tr * 4 + q) * N + ti * F64 + tc * 4) =
          *reinterpret_cast<const int4 *>(&As[tr * 4 + q][tc * 4]);
  };
  if (blockIdx.x == 0 && T > 0) {
    f64i_load(As, M, N, 0, 0);
    __syncthreads();
    close_tile();
    store_tile(0);
  }
  grid.sync();
  for (int k = 0; k < T; ++k) {
    if (blockIdx.x < T - 1) {
      __syncthreads();
      f64i_load(As, M, N, k, k);
      __syncthreads();
    }
    for (int jt = blockIdx.x; jt < T - 1; jt += gridDim.x) {   // phase 2: pivot-row tiles, with transposes
      const int j = jt < k ? jt : jt + 1;
      __syncthreads();
      f64i_load(Bs, M, N, k, j);
      __syncthreads();
      int32_t c[4][4];
#pragma unroll
      for (int q = 0; q < 4; ++q)
#pragma unroll
        for (int jj = 0; jj < 4; ++jj) c[q][jj] = Bs[tr * 4 + q][tc * 4 + jj];
      f64i_mp(As, Bs, c);
      f64i_store(M, N, k, j, c, true);
    }
    grid.sync();
    if (blockIdx.x == 0 && k + 1 < T) {   // lookahead: the next pivot tile updated and closed by block 0
      __syncthreads();
      f64i_load(Bs, M, N, k, k + 1);
      f64i_load(As, M, N, k + 1, k + 1);
      __syncthreads();
      int32_t c[4][4];
#pragma unroll
      for (int q = 0; q < 4; ++q)
#pragma unroll
        for (int jj = 0; jj < 4; ++jj) c[q][jj] = As[tr * 4 + q][tc * 4 + jj];
      f64i_mp(Bs, Bs, c);
      __syncthreads();
#pragma unroll
      for (int q = 0; q < 4; ++q) *reinterpret_cast<int4 *>(&As[tr * 4 + q][tc * 4]) = make_int4(c[q][0], c[q][1], c[q][2], c[q][3]);
      __syncthreads();
      close_tile();
      store_tile(k + 1);
    }
    const int64_t nt = (int64_t)T * (T + 1) / 2;
    const int64_t skip = (int64_t)(k + 1) * (k + 2) / 2 + (k + 1);
    const int gb = gridDim.x > 1 ? (int)gridDim.x - 1 : 1;
    for (int64_t e = gridDim.x > 1 ? blockIdx.x - 1 : 0; e < nt && (gridDim.x == 1 || blockIdx.x > 0); e += gb) {
      if (k + 1 < T && e == skip) continue;
      int i = (int)((sqrt(8.0 * (double)e + 1.0) - 1.0) / 2.0);
      while ((int64_t)(i + 1) * (i + 2) / 2 <= e) ++i;
      while ((int64_t)i * (i + 1) / 2 > e) --i;
      const int jj = i, ii = (int)(e - (int64_t)i * (i + 1) / 2);
      if (ii == k || jj == k) continue;
      __syncthreads();
      f64i_load(As, M, N, k, ii);
      f64i_load(Bs, M, N, k, jj);
      __syncthreads();
      int32_t c[4][4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int4 x = *reinterpret_cast<const int4 *>(M + (int64_t)(ii * F64 + tr * 4 + q) * N + jj * F64 + tc * 4);
        c[q][0] = x.x, c[q][1] = x.y, c[q][2] = x.z, c[q][3] = x.w;
      }
      f64i_mp(As, Bs, c);
      f64i_store(M, N, ii, jj, c, ii != jj);
    }
    grid.sync();
  }
}

__global__ void k_b16_fill(uint16_t *M, int32_t N) {
  const int64_t tot = (int64_t)N * N;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x)
    M[e] = (e / N == e % N) ? 0 : (uint16_t)PC16;
}
__global__ void k_b16_clique(const uint16_t *__restrict__ LR, const int32_t *__restrict__ bcnt,
                             const int32_t *__restrict__ boff, uint16_t *M, int32_t N) {
  const int i = blockIdx.x;
  const int nb = bcnt[i], b0 = boff[i];
  const uint16_t *L = LR + (size_t)i * PCAP * PCAP;
  for (int e = threadIdx.x; e < nb * nb; e += blockDim.x) {
    const int a = e / nb, b = e % nb;
    M[(int64_t)(b0 + a) * N + b0 + b] = (uint16_t)min((uint32_t)L[a * PCAP + b], PC16);
  }
}
__global__ void k_b16_cross(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                            const int32_t *__restrict__ w, const int32_t *__restrict__ bvert, int32_t NB,
                            const int32_t *__restrict__ reg, const int32_t *__restrict__ gidx, uint16_t *M, int32_t N) {
  for (int32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < NB; g += gridDim.x * blockDim.x) {
    const int32_t v = bvert[g], rv = reg[v];
    for (int32_t a = rowptr[v], e = rowptr[v + 1]; a < e; ++a) {
      const int32_t x = col[a];
      if (reg[x] != rv) M[(int64_t)g * N + gidx[x]] = (uint16_t)min(w[a], (int32_t)PC16);   // one arc per pair
    }
  }
}
// capped FW result -> dB16 (0xFFFF = INF), its largest finite entry; *bad when a connected pair reached the cap
__global__ void k_b16_narrow(const uint16_t *__restrict__ M, int32_t N, const int32_t *__restrict__ bvert,
                             const int32_t *__restrict__ cc, int32_t NB, int32_t NBp, uint16_t *dB16, int32_t *stats,
                             int32_t *bad) {
  const int64_t tot = (int64_t)NB * NBp;
  int mx = 0, b = 0;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t g = (int32_t)(e / NBp), h = (int32_t)(e % NBp);
    uint16_t y = 0xFFFF;
    if (h < NB) {
      const uint32_t x = M[(int64_t)g * N + h];
      if (x < PC16) {
        y = (uint16_t)x;
        mx = max(mx, (int)x);
      } else if (cc[bvert[g]] == cc[bvert[h]]) {
        b = 1;
      }
    }
    dB16[e] = y;
  }
  for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(stats, mx);
  if (__syncthreads_or(b) && threadIdx.x == 0) *bad = 1;
}

// rows a caller's output row range [rb, re) of G needs from D (Phase III stages them): the terminal's own
// row, or both ends of a chain vertex; then the regions that hold one
__global__ void k_need_rows(const VDesc *__restrict__ desc, int32_t rb, int32_t re, int32_t *need) {
  for (int32_t s = rb + blockIdx.x * blockDim.x + threadIdx.x; s < re; s += gridDim.x * blockDim.x) {
    const VDesc d = desc[s];
    need[d.p] = 1;
    need[d.q] = 1;
  }
}
__global__ void k_need_regions(const int32_t *__restrict__ need, const int32_t *__restrict__ reg, int32_t n,
                               int32_t *rneed) {
  for (int32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x)
    if (need[v]) rneed[reg[v]] = 1;
}

// int32 D (Np x Np, INF, padding isolated) from the u16 rows
__global__ void k_widen(const uint16_t *__restrict__ D16, int64_t ld16, int32_t nr, int32_t *D, int64_t ldd,
                        int32_t Np) {
  const int64_t tot = (int64_t)Np * Np;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(e / Np), c = (int32_t)(e % Np);
    int32_t x;
    if (r < nr && c < nr) {
      const uint16_t y = D16[(int64_t)r * ld16 + c];
      x = y == 0xFFFF ? INF : (int32_t)y;
    } else {
      x = r == c ? 0 : INF;
    }
    D[(int64_t)r * ldd + c] = x;
  }
}

struct Tmp {
  cudaStream_t st;
  std::vector<void *> ptrs;
  explicit Tmp(cudaStream_t s) : st(s) {}
  ~Tmp() {
    for (void *p : ptrs) cudaFreeAsync(p, st);
  }
  template <typename T>
  bool get(T **p, size_t n) {
    if (cudaMallocAsync((void **)p, sizeof(T) * std::max<size_t>(n, 1), st) != cudaSuccess) return false;
    ptrs.push_back(*p);
    return true;
  }
};

ear_status_t rb1(void *h, const void *d, size_t bytes, cudaStream_t st, const char *what) {
  Readback rb(st);
  cudaError_t e = rb.get(h, d, bytes);
  if (e == cudaSuccess) e = rb.sync();
  if (e != cudaSuccess) {
    set_error("%s: %s", what, cudaGetErrorString(e));
    return EAR_ECUDA;
  }
  return EAR_OK;
}

}  // namespace

void part_free(ear_part_s *q, cudaStream_t st) {
  if (!q) return;
  void *a[] = {q->reg, q->loc, q->perm, q->roff, q->bcnt, q->boff, q->rcomp, q->bvert, q->gidx, q->big, q->vrange};
  for (void *x : a)
    if (x) cudaFreeAsync(x, st);
  delete q;
}

// The partition of a graph into regions (G^r: cached in the plan; the boundary graph: per solve).
ear_status_t part_build(const GView &gv, cudaStream_t st, ear_part_s **out) {
  NvtxRange nvtx_("ear: regions");
  *out = nullptr;
  const int32_t n = gv.n;
  const int32_t *rowptr = gv.rowptr, *col = gv.col, *cc = gv.cc;
  Tmp t(st);
  int32_t *lab[2], *grp, *cnt, *flags, *rid, *gpos, *fstart, *fbnd, *vals;
  uint32_t *keys, *skeys;
  constexpr int NFLAGS = 64;   // [0..15] labelling, [16..23] region totals
  if (!t.get(&lab[0], n) || !t.get(&lab[1], n) || !t.get(&grp, n) || !t.get(&cnt, n) || !t.get(&flags, NFLAGS) ||
      !t.get(&rid, n) || !t.get(&gpos, n) || !t.get(&fstart, n) || !t.get(&fbnd, n) || !t.get(&vals, n) ||
      !t.get(&keys, n) || !t.get(&skeys, n)) {
    set_error("part_prepare: out of device memory");
    return EAR_ENOMEM;
  }
  ear_part_s *q = new ear_part_s();
  auto fail = [&](ear_status_t s) {
    part_free(q, st);
    return s;
  };
  const int g = grid_n(n);
  LabTrace tr(st, -1);
  {
    int per_sm = 0;
    EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_partition, NT, 0));
    const int gc = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, NT), (int64_t)per_sm * num_sms()));
    EAR_CUDA_TRY(dev_memset(flags, 0, 16 * sizeof(int32_t), st));
    static const int32_t pseed = [] {   // lab knob: EAR_PSEED (seed spacing of the first Voronoi pass)
      const char *e = getenv("EAR_PSEED");
      return e ? std::max(2, atoi(e)) : PSEED;
    }();
    int32_t S = pseed;
    void *args[] = {(void *)&rowptr, (void *)&col, (void *)&cc, (void *)&n, (void *)&S, (void *)&lab[0], (void *)&lab[1],
                    (void *)&grp, (void *)&cnt, (void *)&flags};
    count_launch();
    if (cudaLaunchCooperativeKernel((const void *)k_partition, gc, NT, args, 0, st) != cudaSuccess) {
      cudaGetLastError();
      set_error("part_prepare: cooperative launch refused");
      return fail(EAR_EUNSUPPORTED);   // the route does not apply (part_rows: another route runs)
    }
  }
  const int cur = 0;
  tr.mark("build: bfs+split");
  // members by (region, boundary first, id)
  EAR_LAUNCH(k_keys, g, NT, 0, st)(rowptr, col, n, lab[cur], keys, vals);
  if (cudaMallocAsync((void **)&q->perm, sizeof(int32_t) * n, st) != cudaSuccess)
    return fail((set_error("part_prepare: out of device memory"), EAR_ENOMEM));
  int bits = 1;
  while ((int64_t)1 << bits < 2 * (int64_t)n) ++bits;
  size_t tb1 = 0, tb2 = 0, tb3 = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, tb1, keys, skeys, vals, q->perm, n, 0, bits, st);
  cub::DeviceScan::InclusiveSum(nullptr, tb2, fstart, rid, n, st);
  cub::DeviceScan::ExclusiveSum(nullptr, tb3, fbnd, gpos, n, st);
  void *tmp = nullptr;
  if (!t.get((char **)&tmp, std::max({tb1, tb2, tb3})))
    return fail((set_error("part_prepare: out of device memory"), EAR_ENOMEM));
  EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb1, keys, skeys, vals, q->perm, n, 0, bits, st));
  EAR_LAUNCH(k_flags, g, NT, 0, st)(skeys, n, fstart, fbnd);
  EAR_CUDA_TRY(cub::DeviceScan::InclusiveSum(tmp, tb2, fstart, rid, n, st));
  EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb3, fbnd, gpos, n, st));
  // region count K <= n; allocate the per-region arrays for n (small) and fill
  auto need = [&](int32_t **x, size_t m) { return cudaMallocAsync((void **)x, sizeof(int32_t) * std::max<size_t>(m, 1), st); };
  if (need(&q->reg, n) || need(&q->loc, n) || need(&q->gidx, n) || need(&q->roff, (size_t)n + 1) ||
      need(&q->boff, n) || need(&q->bcnt, n) || need(&q->rcomp, n) || need(&q->bvert, n))
    return fail((set_error("part_prepare: out of device memory"), EAR_ENOMEM));
  if (need(&q->big, n) || cudaMallocAsync((void **)&q->vrange, sizeof(int2) * n, st) != cudaSuccess)
    return fail((set_error("part_prepare: out of device memory"), EAR_ENOMEM));
  EAR_CUDA_TRY(dev_memset(q->bcnt, 0, sizeof(int32_t) * n, st));
  int32_t *tot = flags + 16;   // K, NB, max region, max |B_i|, multi, nbig, sum |R_i||B_i| (u64)
  EAR_CUDA_TRY(dev_memset(tot, 0, 8 * sizeof(int32_t), st));
  EAR_LAUNCH(k_fill, g, NT, 0, st)(q->perm, fstart, fbnd, rid, gpos, cc, n, q->reg, q->gidx, q->roff, q->boff, q->bcnt,
                                   q->rcomp, q->bvert, tot);
  EAR_LAUNCH(k_loc, g, NT, 0, st)(q->perm, rid, q->roff, n, q->loc, tot + 2);
  EAR_LAUNCH(k_region_stats, g, NT, 0, st)(q->perm, q->roff, q->bcnt, q->rcomp, tot, q->big, q->vrange);
  int32_t h[24];
  {
    ear_status_t s = rb1(h, flags, sizeof(h), st, "part_prepare");
    if (s != EAR_OK) return fail(s);
  }
  if (h[0]) return fail((set_error("part_prepare: unlabelled vertex after the BFS"), EAR_ECUDA));
  if (h[2]) return fail((set_error("part_prepare: region labelling did not converge"), EAR_ECUDA));
  q->passes = h[1];
  q->K = h[16];
  q->NB = h[17];
  q->max_region = h[18];
  q->max_bnd = h[19];
  q->multi = h[20];
  q->nbig = h[21];
  q->sum_rb = (double)((uint64_t)(uint32_t)h[22] | ((uint64_t)(uint32_t)h[23] << 32));
  q->NBp = (int32_t)round_up(std::max(q->NB, 1), MP_TC);
  tr.mark("build: host lists");
  *out = q;
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

static ear_status_t plan_view(ear_plan_s *p, cudaStream_t st, GView *gv) {
  LabTrace tr(st, -2);
  EAR_TRY(sssp_prepare(p, st));
  tr.mark("view: reduced CSR");
  const int32_t *cc = nullptr;
  EAR_TRY(reduced_labels(p, (int32_t)round_up(p->n_reduced, TILE), st, &cc));
  tr.mark("view: components");
  *gv = GView{p->n_reduced, p->r_rowptr, p->r_col, p->r_w, cc};
  return EAR_OK;
}

// EAR_EUNSUPPORTED: no partition on this device (cooperative launches refused); callers fall back
ear_status_t part_prepare(ear_plan_s *p, cudaStream_t st) {
  if (p->part) return EAR_OK;
  if (p->n_reduced <= 0) {
    set_error("part_prepare: empty reduced graph");
    return EAR_EINVAL;
  }
  GView gv;
  EAR_TRY(plan_view(p, st, &gv));
  EAR_TRY(part_build(gv, st, &p->part));
  p->connected = p->part->multi ? 0 : 1;   // every region in one component <=> G^r connected
  return EAR_OK;
}

// Every row of the view's distance matrix as u16 (0xFFFF = INF, row stride ldo >= round_up(n, 8)) into
// out.  depth: nesting level (the boundary graph of a level is solved by the same route when it is big).
// *applied = false when the route does not apply (too many regions, a region distance or a sum that
// could reach 0xFFFF); nothing is written then.  Profiled (PK_PART / PK_PART_MP) at depth 0 only.
ear_status_t part_solve(const GView &gv, ear_part_s *q, uint16_t *out, int64_t ldo, int depth, bool fw32,
                        bool *applied, cudaStream_t st, const int32_t *rneed = nullptr,
                        const std::function<void()> &before_sync = nullptr) {
  *applied = false;
  const int32_t n = gv.n;
  // mostly tiny components (K near n): the (column blocks x regions) product grid would dominate
  if (q->K > n / 16 && (double)q->K * ceil_div(n, MP_TC) > 65536.0) return EAR_OK;
  const int ps = depth == 0 ? prof_begin(PK_PART, st) : -1;
  LabTrace tr(st, depth);
  Tmp t(st);
  uint16_t *LR = nullptr, *dB16 = nullptr, *DBVt = nullptr, *DBV = nullptr;
  int32_t *stats = nullptr;
  const int32_t NB = q->NB, NBp = q->NBp;
  if (!t.get(&LR, (size_t)q->K * PCAP * PCAP) || !t.get(&stats, 4) || !t.get(&dB16, (size_t)std::max(NB, 1) * NBp) ||
      !t.get(&DBVt, (size_t)n * NBp)) {
    set_error("part_solve: out of device memory");
    return EAR_ENOMEM;
  }
  EAR_CUDA_TRY(dev_memset(stats, 0, 4 * sizeof(int32_t), st));
  const int fw_smem = (PCAP * PCAP + 2 * PCAP) * (int)sizeof(uint16_t);
  EAR_CUDA_TRY(smem_attr((const void *)k_region_fw, fw_smem));
  EAR_LAUNCH(k_region_fw, q->K, FW_NT, fw_smem, st)(gv.rowptr, gv.col, gv.w, q->roff, q->perm, q->reg, q->loc, LR,
                                                     stats);
  if (tr.on) fprintf(stderr, "[part d%d] n=%d K=%d NB=%d max_bnd=%d sum_rb=%.0f passes=%d\n", depth, n, q->K, NB,
                     q->max_bnd, q->sum_rb, q->passes);
  tr.mark("region fw");
  // (3): distances between boundary vertices
  if (NB > 0) {
    bool done = false;
    static const int prec_min = [] {   // lab knob: EAR_PREC_MIN
      const char *e = getenv("EAR_PREC_MIN");
      return e ? atoi(e) : PREC_MIN;
    }();
    if (depth < PREC_DEPTH && NB >= prec_min) {
      // the boundary graph H (cliques d_i on every B_i + the joining arcs) by the same route
      Tmp th(st);
      int32_t *hdeg, *hrow, *hcol, *hw, *hcc, *mn;
      size_t tb = 0;
      cub::DeviceScan::ExclusiveSum(nullptr, tb, (int32_t *)nullptr, (int32_t *)nullptr, NB + 1, st);
      void *tmp = nullptr;
      if (!th.get(&hdeg, (size_t)NB + 1) || !th.get(&hrow, (size_t)NB + 1) || !th.get(&hcc, NB) ||
          !th.get(&mn, n) || !th.get((char **)&tmp, tb)) {
        set_error("part_solve: out of device memory");
        return EAR_ENOMEM;
      }
      EAR_LAUNCH(k_h_deg, grid_n(NB + 1), NT, 0, st)(gv.rowptr, gv.col, q->bvert, NB, q->reg, q->bcnt, hdeg);
      EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb, hdeg, hrow, NB + 1, st));
      int32_t arcs = 0;
      EAR_TRY(rb1(&arcs, hrow + NB, sizeof(int32_t), st, "part_solve"));
      if (!th.get(&hcol, arcs) || !th.get(&hw, arcs)) {
        set_error("part_solve: out of device memory");
        return EAR_ENOMEM;
      }
      EAR_LAUNCH(k_h_fill, grid_n(NB), NT, 0, st)(gv.rowptr, gv.col, gv.w, q->bvert, NB, q->reg, q->gidx, q->bcnt, q->boff,
                                                  LR, hrow, hcol, hw);
      EAR_CUDA_TRY(dev_memset(mn, 0x7F, sizeof(int32_t) * n, st));
      EAR_LAUNCH(k_h_cc, grid_n(NB), NT, 0, st)(q->bvert, gv.cc, NB, mn, nullptr);
      EAR_LAUNCH(k_h_cc, grid_n(NB), NT, 0, st)(q->bvert, gv.cc, NB, mn, hcc);
      const GView hv{NB, hrow, hcol, hw, hcc};
      ear_part_s *qh = nullptr;
      tr.mark("H build");
      const ear_status_t sb = part_build(hv, st, &qh);
      if (sb != EAR_OK && sb != EAR_EUNSUPPORTED) return sb;
      if (qh) {   // (no partition on this device: the dense FW below)
        const ear_status_t s = part_solve(hv, qh, dB16, NBp, depth + 1, fw32, &done, st);
        part_free(qh, st);
        EAR_TRY(s);
      }
      tr.mark("H solved");
      if (done) EAR_LAUNCH(k_max16, grid_n((int64_t)NB * NBp / 8), NT, 0, st)(dB16, NB, NBp, NB, stats + 2);
    }
    if (!done && !fw32 && NB <= FW64_MAX) {   // dense, small: the cooperative 64-tile FW (capped u16)
      uint16_t *M = nullptr;
      int32_t *bad = nullptr;
      const int32_t N64 = (int32_t)round_up(NB, F64);
      if (!t.get(&M, (size_t)N64 * N64) || !t.get(&bad, 1)) {
        set_error("part_solve: out of device memory");
        return EAR_ENOMEM;
      }
      EAR_CUDA_TRY(dev_memset(bad, 0, sizeof(int32_t), st));
      EAR_LAUNCH(k_b16_fill, grid_n((int64_t)N64 * N64), NT, 0, st)(M, N64);
      EAR_LAUNCH(k_b16_clique, q->K, NT, 0, st)(LR, q->bcnt, q->boff, M, N64);
      EAR_LAUNCH(k_b16_cross, grid_n(NB), NT, 0, st)(gv.rowptr, gv.col, gv.w, q->bvert, NB, q->reg, q->gidx, M, N64);
      int per_sm = 0;
      EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_fw64, 256, 0));
      {
        int ps = 0;   // the split schedule's kernel must be co-resident with the same grid
        EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ps, k_fw64s, 256, 0));
        per_sm = std::min(per_sm, ps);
      }
      const int T = N64 / F64;
      const int gfw = (int)std::max<int64_t>(1, std::min<int64_t>((int64_t)T * (T + 1) / 2, (int64_t)per_sm * num_sms()));
      int32_t NN = N64;
      void *args[] = {(void *)&M, (void *)&NN};
      count_launch();
      int32_t h_bad = 1;
      const char *se = getenv("EAR_FW64_SPLIT");   // the split-barrier schedule (0: the grid-barrier kernel)
      int *sbar = nullptr;
      const bool split = (!se || atoi(se) != 0) && gfw >= 2 && t.get(&sbar, 2 * (size_t)T + 1);
      cudaError_t le = cudaErrorUnknown;
      if (split) {
        EAR_CUDA_TRY(dev_memset(sbar, 0, sizeof(int) * (2 * (size_t)T + 1), st));
        void *sargs[] = {(void *)&M, (void *)&NN, (void *)&sbar};
        le = cudaLaunchCooperativeKernel((const void *)k_fw64s, gfw, 256, sargs, 0, st);
      } else {
        le = cudaLaunchCooperativeKernel((const void *)k_fw64, gfw, 256, args, 0, st);
      }
      if (le == cudaSuccess) {
        int32_t *st2 = stats + 2;
        EAR_LAUNCH(k_b16_narrow, grid_n((int64_t)NB * NBp), NT, 0, st)(M, N64, q->bvert, gv.cc, NB, NBp, dB16, st2, bad);
        EAR_TRY(rb1(&h_bad, bad, sizeof(int32_t), st, "part_solve"));
      } else {
        cudaGetLastError();   // no cooperative launch here (e.g. the device is shared): the blocked FW below
      }
      if (h_bad) EAR_CUDA_TRY(dev_memset(stats + 2, 0, sizeof(int32_t), st));   // the int32 FW redoes it
      done = !h_bad;
      tr.mark("dense boundary fw64");
    }
    if (!done && NB <= FW64_MAX) {   // dense, small, int32: the cooperative 64-tile FW without a cap
      int32_t *M32 = nullptr;
      const int32_t N64 = (int32_t)round_up(NB, F64);
      if (!t.get(&M32, (size_t)N64 * N64)) {
        set_error("part_solve: out of device memory");
        return EAR_ENOMEM;
      }
      EAR_LAUNCH(k_bnd_fill, grid_n((int64_t)N64 * N64), NT, 0, st)(M32, N64);
      EAR_LAUNCH(k_bnd_clique, q->K, NT, 0, st)(LR, q->bcnt, q->boff, M32, N64);
      EAR_LAUNCH(k_bnd_cross, grid_n(NB), NT, 0, st)(gv.rowptr, gv.col, gv.w, q->bvert, NB, q->reg, q->gidx, M32, N64);
      int per_sm = 0;
      EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_fw64i, 256, 0));
      const int T = N64 / F64;
      const int gfw = (int)std::max<int64_t>(1, std::min<int64_t>((int64_t)T * (T + 1) / 2, (int64_t)per_sm * num_sms()));
      int32_t NN = N64;
      void *args[] = {(void *)&M32, (void *)&NN};
      count_launch();
      if (cudaLaunchCooperativeKernel((const void *)k_fw64i, gfw, 256, args, 0, st) == cudaSuccess) {
        EAR_LAUNCH(k_bnd_narrow, grid_n((int64_t)NB * NBp / 2), NT, 0, st)(M32, N64, NB, NBp, dB16, stats + 2);
        done = true;
      } else {
        cudaGetLastError();
      }
      tr.mark("dense boundary fw64 int32");
    }
    if (!done) {   // dense: blocked FW over the boundary matrix
      int32_t *dB = nullptr, *labB = nullptr;
      const int32_t NpB = (int32_t)round_up(NB, TILE);
      if (!t.get(&dB, (size_t)NpB * NpB) || !t.get(&labB, NpB)) {
        set_error("part_solve: out of device memory");
        return EAR_ENOMEM;
      }
      EAR_LAUNCH(k_bnd_fill, grid_n((int64_t)NpB * NpB), NT, 0, st)(dB, NpB);
      EAR_LAUNCH(k_bnd_clique, q->K, NT, 0, st)(LR, q->bcnt, q->boff, dB, NpB);
      EAR_LAUNCH(k_bnd_cross, grid_n(NB), NT, 0, st)(gv.rowptr, gv.col, gv.w, q->bvert, NB, q->reg, q->gidx, dB, NpB);
      EAR_LAUNCH(k_bnd_lab, grid_n(NpB), NT, 0, st)(q->bvert, gv.cc, NB, NpB, labB);
      EAR_TRY(fw_single(dB, NpB, NpB, st, labB, NB, !fw32, nullptr));
      EAR_LAUNCH(k_bnd_narrow, grid_n((int64_t)NB * NBp / 2), NT, 0, st)(dB, NpB, NB, NBp, dB16, stats + 2);
      tr.mark("dense boundary fw");
    }
  }
  // the products, each guarded on the device by its no-wrap condition (stats: Lmax, region overflow, max
  // of dB, max of DBV); one readback at the end decides whether the route applied
  if (ps >= 0) prof_end(ps, st, 0);
  const int32_t *cc = q->multi ? gv.cc : nullptr;
  const int pm = depth == 0 ? prof_begin(PK_PART_MP, st) : -1;
  const int64_t ldv = round_up(n, 8);
  int32_t *items = nullptr;
  if (!t.get(&items, (size_t)q->K + 1)) {
    set_error("part_solve: out of device memory");
    return EAR_ENOMEM;
  }
  EAR_CUDA_TRY(smem_attr((const void *)k_region_prod<false>, FINAL_SMEM));
  EAR_CUDA_TRY(smem_attr((const void *)k_region_prod<true>, FINAL_SMEM));
  if (NB > 0) {
    EAR_LAUNCH(k_items, 1, 1024, 0, st)(q->roff, q->bcnt, q->K, NB, nullptr, items);
    EAR_LAUNCH(k_region_prod<false>, PR_MIN * num_sms(), PR_NT, FINAL_SMEM, st)(
        LR, q->roff, q->bcnt, q->boff, q->perm, dB16, NBp, NB, DBVt, NBp, q->reg, q->loc, cc, q->rcomp, q->vrange,
        q->multi, items, q->K, stats);
    if (q->nbig > 0) {
      dim3 g1(NBp / MP_TC, q->nbig);
      EAR_LAUNCH(k_region_mp<false>, g1, MP_NT, 0, st)(LR, q->roff, q->bcnt, q->boff, q->perm, dB16, NBp, NBp, DBVt,
                                                        NBp, q->reg, q->loc, cc, q->rcomp, q->multi, q->big, stats,
                                                        nullptr);
    }
    if (!t.get(&DBV, (size_t)NB * ldv)) {
      set_error("part_solve: out of device memory");
      return EAR_ENOMEM;
    }
    dim3 gt((unsigned)ceil_div(NB, TR), (unsigned)ceil_div(n, TR));
    EAR_LAUNCH(k_transpose16, gt, NT, 0, st)(DBVt, NBp, n, NB, DBV, ldv, stats + 3);
  }
  tr.mark("product1+T");
  EAR_LAUNCH(k_items, 1, 1024, 0, st)(q->roff, q->bcnt, q->K, n, rneed, items);
  EAR_LAUNCH(k_region_prod<true>, PR_MIN * num_sms(), PR_NT, FINAL_SMEM, st)(
      LR, q->roff, q->bcnt, q->boff, q->perm, DBV, ldv, n, out, ldo, q->reg, q->loc, cc, q->rcomp, q->vrange,
      q->multi, items, q->K, stats);
  if (q->nbig > 0) {
    dim3 g2((unsigned)ceil_div(ldo, MP_TC), q->nbig);
    EAR_LAUNCH(k_region_mp<true>, g2, MP_NT, 0, st)(LR, q->roff, q->bcnt, q->boff, q->perm, DBVt, NBp, n, out, ldo,
                                                     q->reg, q->loc, cc, q->rcomp, q->multi, q->big, stats, rneed);
  }
  if (pm >= 0) prof_end(pm, st, (double)n * q->sum_rb + (double)NB * q->sum_rb);
  if (before_sync) before_sync();   // the caller's host work overlaps the products
  int32_t h[4];
  EAR_TRY(rb1(h, stats, sizeof(h), st, "part_solve"));
  tr.mark("final product");
  EAR_CUDA_TRY(cudaGetLastError());
  *applied = !h[1] && h[0] + h[2] < 0xFFFF && h[0] + h[3] < 0xFFFF;
  return EAR_OK;
}

// Every row of D (reduced vertex order) as u16 (0xFFFF = INF, stride ld16 >= round_up(N_r, 8)), or
// -- with D (int32, Np x Np, ldd) -- widened into it.  *applied = false when the route does not apply.
ear_status_t part_rows(ear_plan_s *p, uint16_t *D16, int64_t ld16, int32_t *D, int64_t ldd, int32_t Np, bool *applied,
                       cudaStream_t st, int32_t row_begin, int32_t row_end, const std::function<void()> &before_sync) {
  NvtxRange nvtx_("ear: Phase II by regions");
  *applied = false;
  const int32_t n = p->n_reduced;
  if (n <= 0) return EAR_OK;
  {
    const ear_status_t s = part_prepare(p, st);
    if (s == EAR_EUNSUPPORTED) return EAR_OK;   // not applied: the caller's next route runs
    EAR_TRY(s);
  }
  GView gv;
  EAR_TRY(plan_view(p, st, &gv));
  Tmp t(st);
  uint16_t *out = D16;
  int64_t ldo = ld16;
  if (!out) {
    ldo = round_up(n, 8);
    if (!t.get(&out, (size_t)n * ldo)) {
      set_error("part_rows: out of device memory");
      return EAR_ENOMEM;
    }
  }
  int32_t *rneed = nullptr;   // a strict sub-range of G's rows: only the regions Phase III will stage
  if (!D && (row_begin > 0 || row_end < p->n) && row_end > row_begin) {
    int32_t *need = nullptr;
    if (!t.get(&need, n) || !t.get(&rneed, p->part->K)) {
      set_error("part_rows: out of device memory");
      return EAR_ENOMEM;
    }
    EAR_CUDA_TRY(dev_memset(need, 0, sizeof(int32_t) * n, st));
    EAR_CUDA_TRY(dev_memset(rneed, 0, sizeof(int32_t) * p->part->K, st));
    EAR_LAUNCH(k_need_rows, grid_n(row_end - row_begin), NT, 0, st)(p->desc, row_begin, row_end, need);
    EAR_LAUNCH(k_need_regions, grid_n(n), NT, 0, st)(need, p->part->reg, n, rneed);
  }
  EAR_TRY(part_solve(gv, p->part, out, ldo, 0, (p->flags & EAR_FLAG_FW32) != 0, applied, st, rneed, before_sync));
  if (*applied && D) EAR_LAUNCH(k_widen, grid_n((int64_t)Np * Np), NT, 0, st)(out, ldo, n, D, ldd, Np);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

}  // namespace ear

extern "C" ear_status_t ear_part_info(ear_plan_t p, ear_part_info_t *info) {
  using namespace ear;
  if (!p || !info) {
    set_error("ear_part_info: NULL argument");
    return EAR_EINVAL;
  }
  EAR_TRY(part_prepare(p, p->stream));
  const ear_part_s *q = p->part;
  info->n_regions = q->K;
  info->n_boundary = q->NB;
  info->max_region = q->max_region;
  info->max_boundary = q->max_bnd;
  info->passes = q->passes;
  info->multi_component = q->multi;
  info->sum_region_boundary = q->sum_rb;
  return EAR_OK;
}
