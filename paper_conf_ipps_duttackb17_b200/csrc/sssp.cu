// Phase II alternative: S^r by a single-source shortest-path computation from
// every reduced vertex -- the paper's own Phase II formulation (Alg. 1 lines 4-7: "for each s in
// V(G^r) do DIJKSTRA(G^r, s)") -- instead of the O(N_r^3) blocked FW.  For the sparse
// reduced graphs of the paper's workloads, N_r * M_r * (rounds) << N_r^3.
//
// GPU form: one CTA per source at a time (persistent over sources).  The source's distance row is
// the row of D itself (global, L2-resident while in use); the CTA runs a synchronous label-correcting
// Bellman-Ford over a frontier bitmap in shared memory: every frontier vertex relaxes its arcs with
// atomicMin on the row, improved vertices form the next frontier, until a round improves nothing.
// The fixed point is the exact shortest-path row (integer weights >= 1), identical to the FW result.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"

namespace ear {
namespace {

constexpr int NT = 256;

__global__ void k_r_make_keys(const int32_t *u, const int32_t *v, const int32_t *w, int64_t E, uint64_t *keys,
                              int32_t *vals) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < E; i += (int64_t)gridDim.x * blockDim.x) {
    keys[i] = ((uint64_t)(uint32_t)u[i] << 32) | (uint32_t)v[i];
    vals[i] = w[i];
  }
}

struct MinOp {
  __device__ __forceinline__ int32_t operator()(int32_t a, int32_t b) const { return a < b ? a : b; }
};

__global__ void k_r_split(const uint64_t *keys, int64_t A, int32_t *col, int32_t *deg) {
  for (int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; a < A; a += (int64_t)gridDim.x * blockDim.x) {
    col[a] = (int32_t)(keys[a] & 0xFFFFFFFFu);
    atomicAdd(&deg[keys[a] >> 32], 1);
  }
}

__device__ __forceinline__ int32_t ld_cg(const int32_t *p) { return __ldcg(p); }

// sources: src0 + li, or (with trows) trows[li / 128] * 128 + li % 128; row li of D receives source li
__global__ void __launch_bounds__(NT) k_sssp_bf(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                                               const int32_t *__restrict__ wt, int32_t nr, int32_t Np, int32_t *D,
                                               int64_t ldd, int32_t src0, int32_t nsrc, const int32_t *trows,
                                               unsigned long long *stats) {
  extern __shared__ uint32_t bits[];        // [2][W] frontier bitmaps
  __shared__ int flag[3];
  const int W = (Np + 31) >> 5;
  const int tid = threadIdx.x;
  unsigned long long my_rounds = 0, my_relax = 0, my_improve = 0, my_visits = 0;
  for (int32_t li = blockIdx.x; li < nsrc; li += gridDim.x) {
    const int32_t src = trows ? trows[li >> 7] * TILE + (li & (TILE - 1)) : src0 + li;
    int32_t *dist = D + (int64_t)li * ldd;
    for (int i = tid * 4; i < Np; i += NT * 4)   // Np % 4 == 0, ldd % 4 == 0
      *reinterpret_cast<int4 *>(dist + i) = make_int4(INF, INF, INF, INF);
    for (int w = tid; w < 2 * W; w += NT) bits[w] = 0u;
    if (tid < 3) flag[tid] = 0;
    __syncthreads();
    if (tid == 0) {
      dist[src] = 0;
      bits[src >> 5] = 1u << (src & 31);
    }
    __syncthreads();
    if (src >= nr) continue;   // padding vertex: isolated (INF row, 0 diagonal)
    for (int it = 0;; ++it) {
      uint32_t *cur = bits + (it & 1) * W, *nxt = bits + ((it + 1) & 1) * W;
      if (tid == 0) flag[(it + 1) % 3] = 0;
      for (int w = tid; w < W; w += NT) {
        uint32_t m = cur[w];
        if (!m) continue;
        cur[w] = 0u;   // consumed (this word is owned by this thread in this round)
        while (m) {
          const int b = __ffs(m) - 1;
          m &= m - 1;
          const int v = (w << 5) + b;
          ++my_visits;
          const int32_t dv = ld_cg(dist + v);
          const int a1 = __ldg(rowptr + v + 1);
          for (int a = __ldg(rowptr + v); a < a1; ++a) {
            const int u = __ldg(col + a);
            const int32_t nd = dv + __ldg(wt + a);
            ++my_relax;
            if (nd < ld_cg(dist + u)) {
              const int32_t old = atomicMin(dist + u, nd);
              if (nd < old) {
                ++my_improve;
                atomicOr(&nxt[u >> 5], 1u << (u & 31));
                flag[it % 3] = 1;
              }
            }
          }
        }
      }
      __syncthreads();
      const int more = flag[it % 3];
      ++my_rounds;
      if (!more) break;
    }
    __syncthreads();
  }
  if (stats) {
    if (tid == 0) atomicAdd(&stats[0], my_rounds);
    atomicAdd(&stats[1], my_relax);
    atomicAdd(&stats[2], my_improve);
    atomicAdd(&stats[3], my_visits);
  }
}

// The same label-correcting rounds with the distance row in SHARED memory (Np ints + two bitmaps +
// a frontier list): every read-modify-write of the frontier expansion stays on-chip; the finished row
// is streamed to D with 128-bit stores.  Each round the frontier bitmap is compacted into a list
// (block scan of per-thread popcounts) so that every thread expands about one frontier vertex --
// one dependent (rowptr -> arcs) global-latency chain per round instead of several.  Arcs are packed
// (target, weight) int2 so one load fetches both.
constexpr int SSSP_LIST = 4096;   // frontier list capacity per pass

template <int NTS, int K>
__global__ void __launch_bounds__(NTS) k_sssp_smem(const int32_t *__restrict__ rowptr, const int2 *__restrict__ arcs,
                                                   int32_t nr, int32_t Np, int32_t *D, int64_t ldd,
                                                   int32_t src0, int32_t nsrc, const int32_t *trows,
                                                   unsigned long long *stats) {
  extern __shared__ __align__(16) int32_t sm[];
  int32_t *dist = sm;                                                 // [Np]
  int32_t *list = sm + Np;                                            // [SSSP_LIST]
  uint32_t *bits = reinterpret_cast<uint32_t *>(sm + Np + SSSP_LIST); // [2][W]
  __shared__ int flag[3];
  __shared__ int wsum[NTS / 32];
  const int W = (Np + 31) >> 5;
  const int KW = (W + NTS - 1) / NTS;       // bitmap words per thread (contiguous)
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  unsigned long long my_rounds = 0, my_relax = 0;
  for (int32_t li = blockIdx.x; li < nsrc; li += gridDim.x) {
    const int32_t src = trows ? trows[li >> 7] * TILE + (li & (TILE - 1)) : src0 + li;
    for (int i = tid; i < Np; i += NTS) dist[i] = INF;
    for (int w = tid; w < 2 * W; w += NTS) bits[w] = 0u;
    if (tid < 3) flag[tid] = 0;
    __syncthreads();
    if (tid == 0) {
      dist[src] = 0;
      bits[src >> 5] = 1u << (src & 31);
    }
    __syncthreads();
    if (src < nr) {
      for (int it = 0;; ++it) {
        uint32_t *cur = bits + (it & 1) * W, *nxt = bits + ((it + 1) & 1) * W;
        if (tid == 0) flag[(it + 1) % 3] = 0;
        // 1. rank the frontier: per-thread popcount over its words, block exclusive scan
        const int w0 = tid * KW, w1 = min(W, w0 + KW);
        int cnt = 0;
        for (int w = w0; w < w1; ++w) cnt += __popc(cur[w]);
        int x = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(0xffffffffu, x, o);
          if (lane >= o) x += y;
        }
        if (lane == 31) wsum[warp] = x;
        __syncthreads();
        if (warp == 0) {
          int v = lane < NTS / 32 ? wsum[lane] : 0;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o) v += y;
          }
          if (lane < NTS / 32) wsum[lane] = v;
        }
        __syncthreads();
        const int excl = x - cnt + (warp ? wsum[warp - 1] : 0);
        const int F = wsum[NTS / 32 - 1];
        // 2. expand the frontier pass by pass (list capacity SSSP_LIST)
        for (int base = 0; base < F; base += SSSP_LIST) {
          if (excl < base + SSSP_LIST && excl + cnt > base) {
            int r = excl;
            for (int w = w0; w < w1; ++w) {
              uint32_t m = cur[w];
              while (m) {
                const int b = __ffs(m) - 1;
                m &= m - 1;
                if (r >= base && r < base + SSSP_LIST) list[r - base] = (w << 5) + b;
                ++r;
              }
            }
          }
          __syncthreads();
          const int nb = min(SSSP_LIST, F - base);
          if constexpr (K > 0) {
            // ELL adjacency: vertex v's arcs are the K int2 at arcs[v*K ...] (weight INF padding), so
            // all of a thread's vertices' arcs are fetched with independent 128-bit loads at once
            constexpr int J = 4;   // vertices per thread per batch
            for (int i0 = 0; i0 < nb; i0 += J * NTS) {
              int vv[J];
              int4 e[J][K > 0 ? K / 2 : 1];
#pragma unroll
              for (int j = 0; j < J; ++j) {
                const int i = i0 + j * NTS + tid;
                vv[j] = i < nb ? list[i] : -1;
                const int4 *row = reinterpret_cast<const int4 *>(arcs + (int64_t)max(vv[j], 0) * K);
#pragma unroll
                for (int k = 0; k < K / 2; ++k)
                  e[j][k] = vv[j] >= 0 ? __ldg(row + k) : make_int4(0, INF, 0, INF);
              }
#pragma unroll
              for (int j = 0; j < J; ++j) {
                if (vv[j] < 0) continue;
                const int32_t dv = dist[vv[j]];
#pragma unroll
                for (int k = 0; k < K; ++k) {
                  const int u = (k & 1) ? e[j][k / 2].z : e[j][k / 2].x;
                  const int32_t nd = dv + ((k & 1) ? e[j][k / 2].w : e[j][k / 2].y);
                  if (nd < dist[u]) {
                    if (stats) ++my_relax;
                    const int32_t old = atomicMin(dist + u, nd);
                    if (nd < old) {
                      atomicOr(&nxt[u >> 5], 1u << (u & 31));
                      flag[it % 3] = 1;
                    }
                  }
                }
              }
            }
          } else {
            for (int i = tid; i < nb; i += NTS) {
              const int v = list[i];
              const int32_t dv = dist[v];
              const int a0 = __ldg(rowptr + v), a1 = __ldg(rowptr + v + 1);
              for (int a = a0; a < a1; a += 4) {   // up to 4 independent arc loads in flight
                int2 e[4];
  #pragma unroll
                for (int k = 0; k < 4; ++k) e[k] = (a + k < a1) ? __ldg(arcs + a + k) : make_int2(0, INF);
  #pragma unroll
                for (int k = 0; k < 4; ++k) {
                  if (a + k < a1) {
                    const int u = e[k].x;
                    const int32_t nd = dv + e[k].y;
                    if (stats) ++my_relax;
                    if (nd < dist[u]) {
                      const int32_t old = atomicMin(dist + u, nd);
                      if (nd < old) {
                        atomicOr(&nxt[u >> 5], 1u << (u & 31));
                        flag[it % 3] = 1;
                      }
                    }
                  }
                }
              }
            }
          }
          __syncthreads();
        }
        // 3. the expanded frontier is consumed
        for (int w = w0; w < w1; ++w) cur[w] = 0u;
        const int more = flag[it % 3];
        ++my_rounds;
        if (!more) break;
      }
    }
    __syncthreads();
    int32_t *row = D + (int64_t)li * ldd;
    for (int i = tid * 4; i < Np; i += NTS * 4)   // Np % 4 == 0, 16-byte aligned rows
      *reinterpret_cast<int4 *>(row + i) = *reinterpret_cast<const int4 *>(dist + i);
    __syncthreads();
  }
  if (stats) {
    if (tid == 0) atomicAdd(&stats[0], my_rounds);
    atomicAdd(&stats[1], my_relax);
  }
}

// List-driven rounds with ONE barrier per round (ELL adjacency, K arcs per vertex row).  Round r
// expands list L[r%2] and appends improved vertices to L[(r+1)%2]; membership bitmaps M[.] dedupe the
// appends (set on append, cleared by whoever expands the vertex), and the list counters rotate over
// three slots so that every reset happens in a round where nobody reads or appends that slot.  If a
// round's appends exceed the list capacity, the next round falls back to scanning its bitmap.
template <int NTS, int K>
__global__ void __launch_bounds__(NTS) k_sssp_list(const int2 *__restrict__ ell, int32_t nr, int32_t Np, int32_t *D,
                                                   int64_t ldd, int32_t src0, int32_t nsrc, const int32_t *trows, int cap,
                                                   unsigned long long *stats) {
  extern __shared__ __align__(16) int32_t sm[];
  const int W = (Np + 31) >> 5;
  int32_t *dist = sm;                                               // [Np]
  int32_t *L0 = sm + Np;                                            // [cap]
  int32_t *L1 = L0 + cap;                                           // [cap]
  uint32_t *M0 = reinterpret_cast<uint32_t *>(L1 + cap);            // [W]
  uint32_t *M1 = M0 + W;                                            // [W]
  __shared__ int cnt[3], ovf[3];
  const int tid = threadIdx.x;
  unsigned long long my_rounds = 0, my_relax = 0;
  for (int32_t li = blockIdx.x; li < nsrc; li += gridDim.x) {
    const int32_t src = trows ? trows[li >> 7] * TILE + (li & (TILE - 1)) : src0 + li;
    for (int i = tid; i < Np; i += NTS) dist[i] = INF;
    for (int w = tid; w < 2 * W; w += NTS) M0[w] = 0u;
    if (tid < 3) { cnt[tid] = 0; ovf[tid] = 0; }
    __syncthreads();
    if (tid == 0) {
      dist[src] = 0;
      L0[0] = src;
      M0[src >> 5] = 1u << (src & 31);
      cnt[0] = 1;
    }
    __syncthreads();
    if (src < nr) {
      for (int r = 0;; ++r) {
        int32_t *Lc = (r & 1) ? L1 : L0, *Ln = (r & 1) ? L0 : L1;
        uint32_t *Mc = (r & 1) ? M1 : M0, *Mn = (r & 1) ? M0 : M1;
        const int n = cnt[r % 3];
        const bool scan = ovf[r % 3] != 0;
        int *ncnt = &cnt[(r + 1) % 3];
        int *novf = &ovf[(r + 1) % 3];
        if (tid == 0) { cnt[(r + 2) % 3] = 0; ovf[(r + 2) % 3] = 0; }
        auto relax_from = [&](int v, const int4 *e) {
          const int32_t dv = dist[v];
#pragma unroll
          for (int k = 0; k < K; ++k) {
            const int u = (k & 1) ? e[k / 2].z : e[k / 2].x;
            const int32_t nd = dv + ((k & 1) ? e[k / 2].w : e[k / 2].y);
            if (nd < dist[u]) {
              if (stats) ++my_relax;
              const int32_t old = atomicMin(dist + u, nd);
              if (nd < old) {
                const uint32_t bit = 1u << (u & 31);
                if (!(atomicOr(&Mn[u >> 5], bit) & bit)) {
                  const int idx = atomicAdd(ncnt, 1);
                  if (idx < cap) Ln[idx] = u; else *novf = 1;
                }
              }
            }
          }
        };
        if (!scan) {
          constexpr int J = 4;   // vertices per thread per batch: their arc rows load together
          for (int i0 = 0; i0 < n; i0 += J * NTS) {
            int vv[J];
            int4 e[J][K / 2];
#pragma unroll
            for (int j = 0; j < J; ++j) {
              const int i = i0 + j * NTS + tid;
              vv[j] = i < n ? Lc[i] : -1;
              const int4 *row = reinterpret_cast<const int4 *>(ell + (int64_t)max(vv[j], 0) * K);
#pragma unroll
              for (int k = 0; k < K / 2; ++k) e[j][k] = vv[j] >= 0 ? __ldg(row + k) : make_int4(0, INF, 0, INF);
            }
#pragma unroll
            for (int j = 0; j < J; ++j) {
              if (vv[j] < 0) continue;
              atomicAnd(&Mc[vv[j] >> 5], ~(1u << (vv[j] & 31)));
              relax_from(vv[j], e[j]);
            }
          }
        } else {   // overflowed list: the bitmap holds the frontier
          for (int w = tid; w < W; w += NTS) {
            uint32_t m = Mc[w];
            if (!m) continue;
            atomicAnd(&Mc[w], ~m);
            while (m) {
              const int b = __ffs(m) - 1;
              m &= m - 1;
              const int v = (w << 5) + b;
              int4 e[K / 2];
              const int4 *row = reinterpret_cast<const int4 *>(ell + (int64_t)v * K);
#pragma unroll
              for (int k = 0; k < K / 2; ++k) e[k] = __ldg(row + k);
              relax_from(v, e);
            }
          }
        }
        __syncthreads();
        ++my_rounds;
        if (cnt[(r + 1) % 3] == 0 && ovf[(r + 1) % 3] == 0) break;
      }
    }
    __syncthreads();
    int32_t *row = D + (int64_t)li * ldd;
    for (int i = tid * 4; i < Np; i += NTS * 4)   // Np % 4 == 0, 16-byte aligned rows
      *reinterpret_cast<int4 *>(row + i) = *reinterpret_cast<const int4 *>(dist + i);
    __syncthreads();
  }
  if (stats) {
    if (tid == 0) atomicAdd(&stats[0], my_rounds);
    atomicAdd(&stats[1], my_relax);
  }
}

// ---- the u16 route: distances below 0xFFFF, N_r < 0xFFFF (cfg1-cfg4 of the paper's workloads).
// One CTA per source at a time (persistent, sources from a counter), the distance row in shared memory
// as DistT: u16 (half the bytes: more sources per SM; 16-bit CAS relaxations) or u32 (one ATOMS.MIN per
// relaxation).  One barrier per round: round r expands the list of round r and appends improved
// vertices to round r+1's, deduped by the bitmap M[(r+1)%2] (round r+1 zeroes it while it expands: sets
// and clears of a bitmap are a barrier apart, so no fence is needed -- a vertex improved before its own
// expansion in the same round is expanded once more next round, harmlessly).
// Work is counted in warp instructions (ncu: the kernel is issue-bound), so: the list is cut into
// 32-entry tasks and only warps holding a task run; a warp walks its vertices' ELL slots only while
// some lane still has a real arc (padding sits at the row end); the lists are split into one segment
// per warp and appended WARP-SYNCHRONOUSLY -- after each slot the warp ballots its new vertices and
// writes them at a register-held offset (no shared counter: same-address atomics serialise).  A
// segment that overflows makes the next round scan its bitmap instead.  Arcs are ELL rows of K packed
// u32 (target | weight << 16; padding target 0xFFFF).  A candidate >= 0xFFFF for a still-unreached
// vertex marks the source, and a marked source whose row keeps an unreached vertex raises *sat: the
// caller then falls back to int32 (every shortest path's prefixes are below the final distance, so a
// row without unreached vertices is exact).
// shared-memory accesses by 32-bit shared-window address (computed once per kernel): the generic-pointer
// atomics re-derived the window base (S2R + 3 ALU) in every relaxation
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t atoms_cas(uint32_t a, uint32_t cmp, uint32_t val) {
  uint32_t o;
  asm volatile("atom.shared.cas.b32 %0, [%1], %2, %3;" : "=r"(o) : "r"(a), "r"(cmp), "r"(val) : "memory");
  return o;
}
__device__ __forceinline__ uint32_t atoms_or(uint32_t a, uint32_t val) {
  uint32_t o;
  asm volatile("atom.shared.or.b32 %0, [%1], %2;" : "=r"(o) : "r"(a), "r"(val) : "memory");
  return o;
}
__device__ __forceinline__ void reds_or(uint32_t a, uint32_t val) {
  asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(val) : "memory");
}

template <typename DistT>
__device__ __forceinline__ bool sssp_lower(DistT *d, uint32_t nd, uint32_t cur) {
  if constexpr (sizeof(DistT) == 4) {
    return nd < atomicMin(reinterpret_cast<unsigned int *>(d), nd);
  } else {
    for (;;) {
      const uint16_t old = atomicCAS(reinterpret_cast<unsigned short *>(d), (uint16_t)cur, (uint16_t)nd);
      if (old == (uint16_t)cur) return true;
      cur = old;
      if (nd >= cur) return false;
    }
  }
}

template <int NTS, int K, int J, typename DistT, typename OutT>
__global__ void __launch_bounds__(NTS, 768 / NTS) k_sssp16(const uint4 *__restrict__ ell, int32_t nr, int32_t L, OutT *out,
                                               int64_t ldo, int32_t src0, int32_t nsrc, const int32_t *trows, int cap,
                                               uint32_t delta, int32_t *counter, int32_t *sat,
                                               const uint16_t *__restrict__ maxnb, int32_t *done, int32_t *wm,
                                               unsigned long long *stats) {
  constexpr int NW = NTS / 32;
  constexpr uint32_t DINF = sizeof(DistT) == 2 ? 0xFFFFu : 0xFFFFFFFFu;
  extern __shared__ __align__(16) uint32_t smw[];
  const int W = (L + 31) >> 5;
  const int WS = (W + 3) & ~3;                                               // bitmap stride (16-byte rows)
  const int S = cap / NW;                                                    // segment length
  DistT *dist = reinterpret_cast<DistT *>(smw);                              // [L], L % 8 == 0
  uint32_t *Mb = reinterpret_cast<uint32_t *>(dist + L);                     // [2][WS]
  uint32_t *F = Mb + 2 * WS;                                                 // [WS] the far pile
  uint16_t *Lb = reinterpret_cast<uint16_t *>(F + WS);                       // [2][NW][S]
  const uint32_t dist_s = (uint32_t)__cvta_generic_to_shared(dist);
  const uint32_t F_s = (uint32_t)__cvta_generic_to_shared(F);
  __shared__ __align__(16) int scnt[3][NW];
  __shared__ int ovf[3], s_item, s_sat;
  __shared__ uint32_t s_min[NW];
  __shared__ int s_red[NW], s_k;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const int wpt = (W + NTS - 1) / NTS, w0 = tid * wpt, w1 = min(W, w0 + wpt);   // owned bitmap words
  unsigned long long my_rounds = 0, my_relax = 0;
  for (;;) {
    if (tid == 0) s_item = atomicAdd(counter, 1);
    __syncthreads();
    const int32_t li = s_item;
    if (li >= nsrc) break;
    const int32_t src = trows ? trows[li >> 7] * TILE + (li & (TILE - 1)) : src0 + li;
    // D is symmetric (G undirected): with `maxnb`, the rows of the finished prefix [0, kmax) of sources
    // give d(t, src) = D[t][src] exactly.  Those vertices are final; only the ones with a neighbour
    // >= kmax (maxnb[t] >= kmax) can improve the rest, so they seed the search with the source.
    int kmax = 0;
    if (maxnb) {
      if (tid == 0) s_k = *(volatile int32_t *)wm;
      __syncthreads();
      int k = s_k;
      while (k < li) {   // uniform: the first unfinished row at or after the watermark
        const int t = k + tid;
        const bool fin = t < li && *(volatile const int32_t *)(done + t) != 0;
        const int first = __reduce_min_sync(0xFFFFFFFFu, fin ? 0x7FFFFFFF : min(t, li));
        if (lane == 0) s_red[warp] = first;
        __syncthreads();
        int f = 0x7FFFFFFF;
#pragma unroll
        for (int w = 0; w < NW; ++w) f = min(f, s_red[w]);
        __syncthreads();
        if (f != 0x7FFFFFFF) { k = f; break; }
        k += NTS;
      }
      kmax = min(k, li);
      if (tid == 0 && kmax > s_k) atomicMax(wm, kmax);
      __threadfence();   // acquire: the rows of [0, kmax) are read below
    }
    for (int i = tid; i < L * (int)sizeof(DistT) / 16; i += NTS)
      reinterpret_cast<uint4 *>(dist)[i] = make_uint4(~0u, ~0u, ~0u, ~0u);
    for (int w = tid; w < 2 * WS; w += NTS) Mb[w] = 0u;   // both list bitmaps
    if (tid < 3 * NW) (&scnt[0][0])[tid] = 0;
    if (tid < 3) ovf[tid] = 0;
    if (tid == 0) s_sat = 0;
    __syncthreads();
#pragma unroll 4
    for (int t = tid; t < kmax; t += NTS) {   // column src of the finished rows (L2: written by other CTAs)
      const uint32_t x = (uint32_t)__ldcg(out + (int64_t)t * ldo + src);
      dist[t] = (DistT)(x >= 0xFFFFu ? DINF : x);
    }
    __syncthreads();
    // the far pile starts as {src} + the boundary of the known prefix; round 0 is empty and its advance
    // (thr 0 -> smallest seed + delta) lists every seed below the first threshold
    for (int w = w0; w < w1; ++w) {
      uint32_t f = 0u;
      const int t0 = w << 5;
      if (t0 < kmax) {
        const uint4 *mq = reinterpret_cast<const uint4 *>(maxnb + t0);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint4 m4 = __ldg(mq + q);
          const uint32_t mm[4] = {m4.x, m4.y, m4.z, m4.w};
#pragma unroll
          for (int h = 0; h < 8; ++h) {
            const int b = q * 8 + h, t = t0 + b;
            const uint32_t nb = (mm[h >> 1] >> ((h & 1) * 16)) & 0xFFFFu;
            if (t < kmax && nb >= (uint32_t)kmax && dist[t] != (DistT)DINF) f |= 1u << b;
          }
        }
      }
      if ((src >> 5) == w) f |= 1u << (src & 31);
      F[w] = f;
    }
    if (tid == 0) dist[src] = 0;   // a padding source (src >= nr) has no arcs: its row is INF but the diagonal
    __syncthreads();
    if (src < nr) {
      uint32_t thr = 0;   // near-far: only vertices below thr are expanded (uniform)
      int c0 = 0, c1 = 1, c2 = 2, par = 0;   // count slots of rounds r, r+1, r+2 (r % 3 ...) and r & 1
      for (int r = 0;; ++r) {
        const uint16_t *Lc = Lb + par * (NW * S);
        uint16_t *Ln = Lb + (par ^ 1) * (NW * S) + warp * S;   // this warp's segment
        uint32_t *Mc = Mb + par * WS, *Mn = Mb + (par ^ 1) * WS;
        const uint32_t Mn_s = (uint32_t)__cvta_generic_to_shared(Mn);
        const bool scan = ovf[c0] != 0;
        int *ncnt = &scnt[c1][warp];
        int *novf = &ovf[c1];
        if (tid < NW) scnt[c2][tid] = 0;
        if (tid == 0) ovf[c2] = 0;
        int wc = 0;   // warp-uniform append offset into this warp's segment
        // relax arc a from a vertex at distance dv; true when u is new on round r+1's list
        auto relax = [&](uint32_t dv, uint32_t a) -> bool {
          const uint32_t u = a & 0xFFFFu;
          if (u == 0xFFFFu) return false;
          const uint32_t nd = dv + (a >> 16);
          uint32_t cur;
          if constexpr (sizeof(DistT) == 2) {
            // the 32-bit word holding d(u): one LDS, and a CAS on the word (the compiler's 16-bit CAS
            // emulation costs ~22 instructions)
            const uint32_t wa = dist_s + ((u << 1) & ~3u);
            const uint32_t sh = (u & 1u) << 4;
            uint32_t w = lds_u32(wa);
            cur = (w >> sh) & 0xFFFFu;
            if (nd >= 0xFFFFu) {   // not representable: harmless unless u stays unreached
              if (cur == DINF) s_sat = 1;
              return false;
            }
            for (;;) {
              if (nd >= cur) return false;
              const uint32_t prev = atoms_cas(wa, w, w ^ ((cur ^ nd) << sh));
              if (prev == w) break;
              w = prev;
              cur = (w >> sh) & 0xFFFFu;
            }
          } else {
            cur = dist[u];
            if (nd >= 0xFFFFu) {
              if (cur == DINF) s_sat = 1;
              return false;
            }
            if (nd >= cur || !sssp_lower(dist + u, nd, cur)) return false;
          }
          if (stats) ++my_relax;
          const uint32_t bit = 1u << (u & 31);
          if (nd >= thr) {   // far: waits for the threshold
            reds_or(F_s + ((u >> 5) << 2), bit);
            return false;
          }
          return !(atoms_or(Mn_s + ((u >> 5) << 2), bit) & bit);
        };
        if (!scan) {
          int c[NW];
#pragma unroll
          for (int q = 0; q < NW / 4; ++q) {
            const int4 c4 = reinterpret_cast<const int4 *>(scnt[c0])[q];
            c[4 * q] = min(c4.x, S); c[4 * q + 1] = min(c4.y, S); c[4 * q + 2] = min(c4.z, S); c[4 * q + 3] = min(c4.w, S);
          }
          int n = 0;
#pragma unroll
          for (int w = 0; w < NW; ++w) n += c[w];
          const int ntask = (n + 31) >> 5;
          for (int q = tid; q < WS / 4; q += NTS)   // nobody sets Mc this round
            reinterpret_cast<uint4 *>(Mc)[q] = make_uint4(0u, 0u, 0u, 0u);
          // a narrow frontier leaves warps idle: then f warps share each task, warp g taking the ELL
          // groups g and g + f (4 arcs each) -- the slot chain a task warp runs serially gets f times shorter
          int f = 1;
          if (K / 4 > 1)
            while (2 * f <= K / 4 && ntask * 2 * f <= NW) f *= 2;
          int pre[NW + 1];
          pre[0] = 0;
          if (warp < ntask * f) {   // (only warps holding a task look entries up)
#pragma unroll
            for (int w = 0; w < NW; ++w) pre[w + 1] = pre[w] + c[w];
          }
          auto entry = [&](int i) -> int {
            int sg = 0;
#pragma unroll
            for (int w = 1; w < NW; ++w) sg += i >= pre[w];
            return Lc[sg * S + i - pre[sg]];
          };
          if (f > 1) {
            if (warp < ntask * f) {   // warp-uniform
              const int t = warp % ntask, g = warp / ntask, i = t * 32 + lane;
              const int v = i < n ? entry(i) : -1;
              const uint4 *row = ell + (int64_t)max(v, 0) * (K / 4);
              const uint4 pad = make_uint4(~0u, ~0u, ~0u, ~0u);
              const uint4 e0 = v >= 0 ? __ldg(row + g) : pad;
              const uint4 e1 = (v >= 0 && g + f < K / 4) ? __ldg(row + g + f) : pad;
              const uint32_t dv = v >= 0 ? (uint32_t)dist[v] : 0u;
#pragma unroll
              for (int k = 0; k < 8; ++k) {
                const uint4 q = k < 4 ? e0 : e1;
                const uint32_t a = (k & 3) == 0 ? q.x : (k & 3) == 1 ? q.y : (k & 3) == 2 ? q.z : q.w;
                if (!__any_sync(0xFFFFFFFFu, (a & 0xFFFFu) != 0xFFFFu)) break;   // padding from here on
                const bool push = relax(dv, a);
                const unsigned bal = __ballot_sync(0xFFFFFFFFu, push);
                if (push) {
                  const int idx = wc + __popc(bal & lt);
                  if (idx < S) Ln[idx] = (uint16_t)(a & 0xFFFFu);
                }
                wc += __popc(bal);
              }
            }
          } else
          for (int t0 = warp; t0 < ntask; t0 += J * NW) {   // warp-uniform: the ballots see all lanes
            int vv[J];
            uint4 e[J][K / 4];
#pragma unroll
            for (int j = 0; j < J; ++j) {
              const int i = (t0 + j * NW) * 32 + lane;
              vv[j] = i < n ? entry(i) : -1;
              const uint4 *row = ell + (int64_t)max(vv[j], 0) * (K / 4);
#pragma unroll
              for (int k = 0; k < K / 4; ++k) e[j][k] = vv[j] >= 0 ? __ldg(row + k) : make_uint4(~0u, ~0u, ~0u, ~0u);
            }
#pragma unroll
            for (int j = 0; j < J; ++j) {
              if (t0 + j * NW >= ntask) break;
              const uint32_t dv = vv[j] >= 0 ? (uint32_t)dist[vv[j]] : 0u;
#pragma unroll
              for (int k = 0; k < K; ++k) {
                const uint4 q = e[j][k / 4];
                const uint32_t a = (k & 3) == 0 ? q.x : (k & 3) == 1 ? q.y : (k & 3) == 2 ? q.z : q.w;
                if (!__any_sync(0xFFFFFFFFu, (a & 0xFFFFu) != 0xFFFFu)) break;   // padding from here on
                const bool push = relax(dv, a);
                const unsigned bal = __ballot_sync(0xFFFFFFFFu, push);
                if (push) {
                  const int idx = wc + __popc(bal & lt);
                  if (idx < S) Ln[idx] = (uint16_t)(a & 0xFFFFu);
                }
                wc += __popc(bal);
              }
            }
          }
          if (lane == 0) {
            *ncnt = wc;
            if (wc > S) *novf = 1;
          }
        } else {   // an overflowed segment: the bitmap holds every vertex listed for this round
          for (int w = w0; w < w1; ++w) {
            uint32_t m = Mc[w];
            Mc[w] = 0u;
            while (m) {
              const int b = __ffs(m) - 1;
              m &= m - 1;
              const int v = (w << 5) + b;
              uint4 e[K / 4];
#pragma unroll
              for (int k = 0; k < K / 4; ++k) e[k] = __ldg(ell + (int64_t)v * (K / 4) + k);
              const uint32_t dv = dist[v];
#pragma unroll
              for (int k = 0; k < K; ++k) {
                const uint4 q = e[k / 4];
                const uint32_t a = (k & 3) == 0 ? q.x : (k & 3) == 1 ? q.y : (k & 3) == 2 ? q.z : q.w;
                if (relax(dv, a)) {
                  const int idx = atomicAdd(ncnt, 1);
                  if (idx < S) Ln[idx] = (uint16_t)(a & 0xFFFFu); else *novf = 1;
                }
              }
            }
          }
        }
        __syncthreads();
        ++my_rounds;
        int more = ovf[c1];
#pragma unroll
        for (int q = 0; q < NW / 4; ++q) {
          const int4 c4 = reinterpret_cast<const int4 *>(scnt[c1])[q];
          more |= c4.x | c4.y | c4.z | c4.w;
        }
        {   // rotate the slots for round r+1
          const int t = c0;
          c0 = c1; c1 = c2; c2 = t;
          par ^= 1;
        }
        if (more) continue;
        // the near pile is empty: raise the threshold to (smallest live far distance) + delta and list
        // the far vertices below it for round r+1.  A far entry already below the old threshold is stale
        // (a later improvement put it on a near list): it is dropped.
        uint32_t mn = 0xFFFFFFFFu;
        for (int w = w0; w < w1; ++w) {
          uint32_t m = F[w];
          while (m) {
            const int b = __ffs(m) - 1;
            m &= m - 1;
            const uint32_t d = dist[(w << 5) + b];
            if (d >= thr) mn = min(mn, d);
          }
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) mn = min(mn, __shfl_xor_sync(0xFFFFFFFFu, mn, o));
        if (lane == 0) s_min[warp] = mn;
        __syncthreads();
        mn = 0xFFFFFFFFu;
#pragma unroll
        for (int w = 0; w < NW; ++w) mn = min(mn, s_min[w]);
        if (mn == 0xFFFFFFFFu) break;   // no live far vertex: the row is final
        const uint32_t told = thr;
        thr = mn + delta;
        {
          uint32_t *Mn = Mb + par * WS;   // round r+1's list bitmap (owned words: plain stores)
          uint16_t *Ln = Lb + par * (NW * S) + warp * S;
          int wc = 0;
          for (int wb = warp * 32 * wpt; wb < W; wb += NTS * wpt) {   // warp-uniform over the owned words
            for (int q = 0; q < wpt; ++q) {
              const int w = wb + lane * wpt + q;
              uint32_t m = w < W ? F[w] : 0u, take = 0u, stale = 0u;
              for (uint32_t x = m; x; x &= x - 1) {
                const int b = __ffs(x) - 1;
                const uint32_t d = dist[(w << 5) + b];
                if (d < told) stale |= 1u << b;
                else if (d < thr) take |= 1u << b;
              }
              if (w < W) {
                F[w] = m & ~(take | stale);
                Mn[w] |= take;
              }
              while (__any_sync(0xFFFFFFFFu, take != 0u)) {
                const bool has = take != 0u;
                const int b = has ? __ffs(take) - 1 : 0;
                take &= take - 1;
                const unsigned bal = __ballot_sync(0xFFFFFFFFu, has);
                if (has) {
                  const int idx = wc + __popc(bal & lt);
                  if (idx < S) Ln[idx] = (uint16_t)((w << 5) + b);
                }
                wc += __popc(bal);
              }
            }
          }
          if (lane == 0) {
            scnt[c0][warp] = wc;
            if (wc > S) ovf[c0] = 1;
          }
        }
        __syncthreads();
      }
    }
    if (s_sat) {   // uniform (read after the last round's barrier)
      bool un = false;
      for (int i = tid; i < nr; i += NTS) un |= dist[i] == DINF;
      if (__syncthreads_or(un) && tid == 0) atomicOr(sat, 1);
    }
    OutT *row = out + (int64_t)li * ldo;
    for (int i = tid; i < L / 8; i += NTS) {   // 8 entries per step
      uint32_t x[8];
      if constexpr (sizeof(DistT) == 2) {
        const uint4 q = reinterpret_cast<const uint4 *>(dist)[i];
        const uint32_t h[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
        for (int k = 0; k < 4; ++k) { x[2 * k] = h[k] & 0xFFFFu; x[2 * k + 1] = h[k] >> 16; }
      } else {
        const uint4 q0 = reinterpret_cast<const uint4 *>(dist)[2 * i], q1 = reinterpret_cast<const uint4 *>(dist)[2 * i + 1];
        x[0] = q0.x; x[1] = q0.y; x[2] = q0.z; x[3] = q0.w; x[4] = q1.x; x[5] = q1.y; x[6] = q1.z; x[7] = q1.w;
      }
      if constexpr (sizeof(OutT) == 2) {
        uint32_t y[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) y[k] = min(x[2 * k], 0xFFFFu) | (min(x[2 * k + 1], 0xFFFFu) << 16);
        reinterpret_cast<uint4 *>(row)[i] = make_uint4(y[0], y[1], y[2], y[3]);
      } else {
        int32_t y[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) y[k] = x[k] >= 0xFFFFu ? INF : (int32_t)x[k];
        reinterpret_cast<int4 *>(row)[2 * i] = make_int4(y[0], y[1], y[2], y[3]);
        reinterpret_cast<int4 *>(row)[2 * i + 1] = make_int4(y[4], y[5], y[6], y[7]);
      }
    }
    __syncthreads();
    if (maxnb && tid == 0) {   // publish: every thread's row stores precede the flag (barrier + fence)
      __threadfence();
      atomicExch(done + li, 1);
    }
  }
  if (stats) {
    if (tid == 0) atomicAdd(&stats[0], my_rounds);
    atomicAdd(&stats[1], my_relax);
  }
}

__global__ void k_sum_w(const int32_t *w, int32_t A, unsigned long long *sum) {
  unsigned long long t = 0;
  for (int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; a < A; a += (int64_t)gridDim.x * blockDim.x)
    t += (unsigned long long)w[a];
  atomicAdd(sum, t);
}

__global__ void k_maxnb16(const int32_t *rowptr, const int32_t *col, int32_t nr, int32_t len, uint16_t *mx) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < len; v += (int64_t)gridDim.x * blockDim.x) {
    int m = 0;
    if (v < nr)
      for (int a = rowptr[v]; a < rowptr[v + 1]; ++a) m = max(m, col[a]);
    mx[v] = (uint16_t)m;
  }
}

__global__ void k_build_ell16(const int32_t *rowptr, const int32_t *col, const int32_t *w, int32_t nr, int K,
                              uint32_t *ell) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < nr; v += (int64_t)gridDim.x * blockDim.x) {
    const int a0 = rowptr[v], d = rowptr[v + 1] - a0;
    for (int k = 0; k < K; ++k)
      ell[v * K + k] = k < d ? ((uint32_t)col[a0 + k] | ((uint32_t)min(w[a0 + k], 0xFFFF) << 16)) : 0xFFFFFFFFu;
  }
}

__global__ void k_build_ell(const int32_t *rowptr, const int32_t *col, const int32_t *w, int32_t nr, int K,
                            int2 *ell) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < nr; v += (int64_t)gridDim.x * blockDim.x) {
    const int a0 = rowptr[v], d = rowptr[v + 1] - a0;
    for (int k = 0; k < K; ++k) ell[v * K + k] = k < d ? make_int2(col[a0 + k], w[a0 + k]) : make_int2(0, INF);
  }
}

__global__ void k_max_deg(const int32_t *rowptr, int32_t nr, int32_t *out) {
  int m = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < nr; v += (int64_t)gridDim.x * blockDim.x)
    m = max(m, rowptr[v + 1] - rowptr[v]);
  atomicMax(out, m);
}

__global__ void k_pack_arcs(const int32_t *col, const int32_t *w, int32_t A, int2 *arcs) {
  for (int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; a < A; a += (int64_t)gridDim.x * blockDim.x)
    arcs[a] = make_int2(col[a], w[a]);
}

}  // namespace

// Reduced-graph CSR (parallel G^r arcs -> minimum weight), built once per plan.
ear_status_t sssp_prepare(ear_plan_s *p, cudaStream_t st) {
  if (p->r_rowptr) return EAR_OK;
  const int64_t E = p->n_redges;
  const int32_t nr = p->n_reduced;
  uint64_t *k0 = nullptr, *k1 = nullptr, *uk = nullptr;
  int32_t *v0 = nullptr, *v1 = nullptr, *uv = nullptr, *nruns = nullptr, *deg = nullptr;
  void *tmp = nullptr;
  size_t tb1 = 0, tb2 = 0, tb3 = 0;
  const int64_t E1 = std::max<int64_t>(E, 1);
  auto alloc = [&](void **q, size_t b) { return cudaMallocAsync(q, std::max<size_t>(b, 16), st); };
  cudaError_t e = cudaSuccess;
  e = alloc((void **)&k0, 8 * E1); if (e == cudaSuccess) e = alloc((void **)&k1, 8 * E1);
  if (e == cudaSuccess) e = alloc((void **)&uk, 8 * E1);
  if (e == cudaSuccess) e = alloc((void **)&v0, 4 * E1);
  if (e == cudaSuccess) e = alloc((void **)&v1, 4 * E1);
  if (e == cudaSuccess) e = alloc((void **)&uv, 4 * E1);
  if (e == cudaSuccess) e = alloc((void **)&nruns, 4);
  if (e == cudaSuccess) e = alloc((void **)&deg, 4 * ((size_t)nr + 1));
  if (e != cudaSuccess) { set_error("sssp_prepare: %s", cudaGetErrorString(e)); return EAR_ENOMEM; }
  int32_t A = 0;
  if (E > 0) {
    const int g = (int)std::min<int64_t>(ceil_div(E, 256), 4096);
    EAR_LAUNCH(k_r_make_keys, g, 256, 0, st)(p->re_u, p->re_v, p->re_w, E, k0, v0);
    cub::DoubleBuffer<uint64_t> dk(k0, k1);
    cub::DoubleBuffer<int32_t> dv(v0, v1);
    int bits = 1;
    while ((1ll << bits) < nr) ++bits;
    cub::DeviceRadixSort::SortPairs(nullptr, tb1, dk, dv, (int)E, 0, 32 + bits, st);
    cub::DeviceReduce::ReduceByKey(nullptr, tb2, k0, uk, v0, uv, nruns, MinOp(), (int)E, st);
    cub::DeviceScan::ExclusiveSum(nullptr, tb3, deg, deg, nr + 1, st);
    EAR_CUDA_TRY(cudaMallocAsync(&tmp, std::max({tb1, tb2, tb3, (size_t)16}), st));
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb1, dk, dv, (int)E, 0, 32 + bits, st));
    EAR_CUDA_TRY(cub::DeviceReduce::ReduceByKey(tmp, tb2, dk.Current(), uk, dv.Current(), uv, nruns, MinOp(), (int)E,
                                                st));
    Readback rb(st);
    EAR_CUDA_TRY(rb.get(&A, nruns, 4));
    EAR_CUDA_TRY(rb.sync());
  }
  EAR_CUDA_TRY(cudaMallocAsync((void **)&p->r_rowptr, 4 * ((size_t)nr + 1), st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&p->r_col, 4 * (size_t)std::max(A, 1), st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&p->r_w, 4 * (size_t)std::max(A, 1), st));
  EAR_CUDA_TRY(dev_memset(deg, 0, 4 * ((size_t)nr + 1), st));
  if (A > 0) {
    const int g = (int)std::min<int64_t>(ceil_div(A, 256), 4096);
    EAR_LAUNCH(k_r_split, g, 256, 0, st)(uk, A, p->r_col, deg);
    EAR_CUDA_TRY(dev_copy(p->r_w, uv, 4 * (size_t)A, st));
    EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb3, deg, p->r_rowptr, nr + 1, st));
  } else {
    EAR_CUDA_TRY(dev_memset(p->r_rowptr, 0, 4 * ((size_t)nr + 1), st));
  }
  p->n_rarcs = A;
  void *fr[] = {k0, k1, uk, v0, v1, uv, nruns, deg, tmp};
  for (void *q : fr)
    if (q) cudaFreeAsync(q, st);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

template <int NTS, int K>
static ear_status_t sssp_launch(ear_plan_s *p, int32_t *D, int64_t ldd, int32_t Np, int32_t row0, int32_t rows,
                                const int32_t *trows,
                                int smem_s, int nsm, unsigned long long *d_stats, cudaStream_t st) {
  EAR_CUDA_TRY(smem_attr((const void *)k_sssp_smem<NTS, K>, smem_s));
  int per_sm = 1;
  EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_sssp_smem<NTS, K>, NTS, smem_s));
  const int64_t grid = std::min<int64_t>(rows, (int64_t)nsm * std::max(per_sm, 1));
  int s = prof_begin(PK_SSSP, st);
  EAR_LAUNCH((k_sssp_smem<NTS, K>), (unsigned)grid, NTS, smem_s, st)(
      p->r_rowptr, reinterpret_cast<const int2 *>(p->r_arcs), p->n_reduced, Np, D, ldd, row0, rows, trows,
      d_stats);
  prof_end(s, st, (double)rows * (double)p->n_rarcs);
  if (d_stats) {
    unsigned long long h[4];
    EAR_CUDA_TRY(cudaMemcpyAsync(h, d_stats, 32, cudaMemcpyDeviceToHost, st));
    EAR_CUDA_TRY(cudaStreamSynchronize(st));
    fprintf(stderr, "[sssp smem K=%d] grid=%lld per_sm=%d rows=%d rounds=%.1f/source relax=%.0f/source arcs=%d\n", K,
            (long long)grid, per_sm, rows, (double)h[0] / rows, (double)h[1] / rows, p->n_rarcs);
  }
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

template <int NTS, int K>
static ear_status_t sssp_list_launch(ear_plan_s *p, int32_t *D, int64_t ldd, int32_t Np, int32_t row0, int32_t rows,
                                     const int32_t *trows,
                                     int max_smem, int nsm, unsigned long long *d_stats, cudaStream_t st) {
  const int W = (Np + 31) / 32;
  const int fixed = 4 * Np + 8 * W + 64;
  const int cap = std::min(Np, (max_smem - fixed) / 8);
  const int smem = 4 * Np + 8 * cap + 8 * W;
  EAR_CUDA_TRY(smem_attr((const void *)k_sssp_list<NTS, K>, smem));
  int per_sm = 1;
  EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_sssp_list<NTS, K>, NTS, smem));
  const int64_t grid = std::min<int64_t>(rows, (int64_t)nsm * std::max(per_sm, 1));
  int s = prof_begin(PK_SSSP, st);
  EAR_LAUNCH((k_sssp_list<NTS, K>), (unsigned)grid, NTS, smem, st)(
      reinterpret_cast<const int2 *>(p->r_arcs), p->n_reduced, Np, D, ldd, row0, rows, trows, cap, d_stats);
  prof_end(s, st, (double)rows * (double)p->n_rarcs);
  if (d_stats) {
    unsigned long long h[4];
    EAR_CUDA_TRY(cudaMemcpyAsync(h, d_stats, 32, cudaMemcpyDeviceToHost, st));
    EAR_CUDA_TRY(cudaStreamSynchronize(st));
    fprintf(stderr, "[sssp list K=%d cap=%d] grid=%lld per_sm=%d rows=%d rounds=%.1f/source relax=%.0f/source\n", K,
            cap, (long long)grid, per_sm, rows, (double)h[0] / rows, (double)h[1] / rows);
  }
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// ---- u16 route (host side)
static ear_status_t ell16_prepare(ear_plan_s *p, cudaStream_t st) {
  if (p->r_k16 >= 0) return EAR_OK;
  EAR_TRY(sssp_prepare(p, st));
  const int32_t nr = p->n_reduced;
  p->r_k16 = 0;
  if (nr <= 0 || nr >= 0xFFFF) return EAR_OK;
  int32_t *d_md = nullptr, md = 0;
  unsigned long long wsum = 0;
  EAR_CUDA_TRY(cudaMallocAsync((void **)&d_md, 16, st));
  EAR_CUDA_TRY(dev_memset(d_md, 0, 16, st));
  unsigned long long *d_sum = reinterpret_cast<unsigned long long *>(d_md + 2);
  EAR_LAUNCH(k_max_deg, (int)std::min<int64_t>(ceil_div(nr, 256), 4096), 256, 0, st)(p->r_rowptr, nr, d_md);
  if (p->n_rarcs > 0)
    EAR_LAUNCH(k_sum_w, (int)std::min<int64_t>(ceil_div(p->n_rarcs, 256), 1024), 256, 0, st)(p->r_w, p->n_rarcs, d_sum);
  {
    Readback rb(st);
    EAR_CUDA_TRY(rb.get(&md, d_md, 4));
    EAR_CUDA_TRY(rb.get(&wsum, d_sum, 8));
    EAR_CUDA_TRY(rb.sync());
  }
  cudaFreeAsync(d_md, st);
  // near-far step: 16 mean arc weights (cfg4, simulated: 5x fewer improvements than plain rounds at
  // about the same round count; smaller steps trade rounds for work)
  const double mean_w = p->n_rarcs > 0 ? (double)wsum / (double)p->n_rarcs : 1.0;
  p->r_delta = (uint32_t)std::min(65535.0, std::max(1.0, 16.0 * mean_w));
  const int K = md <= 4 ? 4 : md <= 8 ? 8 : md <= 12 ? 12 : md <= 16 ? 16 : 0;
  if (K == 0) return EAR_OK;
  const int32_t lm = (int32_t)round_up(nr, 64);   // read in whole 32-vertex words by the kernel
  EAR_CUDA_TRY(cudaMallocAsync((void **)&p->r_maxnb, sizeof(uint16_t) * (size_t)lm, st));
  EAR_LAUNCH(k_maxnb16, (int)std::min<int64_t>(ceil_div(lm, 256), 4096), 256, 0, st)(p->r_rowptr, p->r_col, nr, lm,
                                                                                   p->r_maxnb);
  EAR_CUDA_TRY(cudaMallocAsync((void **)&p->r_ell16, sizeof(uint32_t) * (size_t)K * nr, st));
  EAR_LAUNCH(k_build_ell16, (int)std::min<int64_t>(ceil_div(nr, 256), 4096), 256, 0, st)(
      p->r_rowptr, p->r_col, p->r_w, nr, K, p->r_ell16);
  p->r_k16 = K;
  return EAR_OK;
}

// 256 threads per source (512 measured slower in every u16 case: idle warps per round)
constexpr int SSSP16_NT = 256;
constexpr int SSSP16_MAX_CTAS = 2048 / SSSP16_NT;
// shared memory of one source: the row (L entries of db bytes), two lists (cap u16 each), three bitmaps
static int sssp16_smem(int L, int cap, int db) { return db * L + 4 * cap + 12 * (((L + 31) / 32 + 3) & ~3); }

template <int NTS, int K, typename DistT, typename OutT>
static ear_status_t sssp16_launch(ear_plan_s *p, OutT *out, int64_t ldo, int32_t L, int32_t row0, int32_t rows,
                                  const int32_t *trows, int cap, int smem, int32_t *ws,
                                  unsigned long long *d_stats, cudaStream_t st) {
  int32_t *counter = ws, *sat = ws + 1, *wm = ws + 2, *done = ws + 4;
  constexpr int J = 2;   // two 32-vertex tasks per warp when the frontier is wide (their ELL loads overlap)
  auto kern = k_sssp16<NTS, K, J, DistT, OutT>;
  EAR_CUDA_TRY(smem_attr((const void *)kern, smem));
  int per_sm = 1;
  EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, NTS, smem));
  const int64_t grid = std::min<int64_t>(rows, (int64_t)num_sms() * std::max(per_sm, 1));
  int s = prof_begin(PK_SSSP, st);
  uint32_t delta = p->r_delta;
  if (const char *e = getenv("EAR_SSSP_DELTA")) delta = atoi(e) > 0 ? (uint32_t)atoi(e) : 0xFFFFFFFFu;   // lab knob
  // row reuse (D symmetric): the single-GPU solve of every row in order -- sources 0.. with row li = source li
  static const bool reuse_off = [] {
    const char *e = getenv("EAR_SSSP_REUSE");   // 0: every source searches the whole graph (A/B)
    return e && atoi(e) == 0;
  }();
  const uint16_t *mx = (!reuse_off && row0 == 0 && !trows) ? p->r_maxnb : nullptr;
  EAR_LAUNCH(kern, (unsigned)grid, NTS, smem, st)(reinterpret_cast<const uint4 *>(p->r_ell16), p->n_reduced, L, out,
                                                  ldo, row0, rows, trows, cap, delta, counter, sat, mx, done, wm,
                                                  d_stats);
  // algorithmic work: one relaxation per arc per (real) source -- Dijkstra's count; padding sources are free
  const int64_t real = trows ? rows : std::max<int64_t>(0, std::min<int64_t>(rows, (int64_t)p->n_reduced - row0));
  prof_end(s, st, (double)real * (double)p->n_rarcs);
  if (d_stats) {
    unsigned long long h[2];
    EAR_CUDA_TRY(cudaMemcpyAsync(h, d_stats, 16, cudaMemcpyDeviceToHost, st));
    EAR_CUDA_TRY(cudaStreamSynchronize(st));
    fprintf(stderr, "[sssp16 NT=%d K=%d dist=u%d cap=%d smem=%d] grid=%lld per_sm=%d rows=%d rounds=%.1f/source improve=%.0f/source\n",
            NTS, K, (int)(8 * sizeof(DistT)), cap, smem, (long long)grid, per_sm, rows, (double)h[0] / rows,
            (double)h[1] / rows);
  }
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

template <int NTS, typename DistT, typename OutT>
static ear_status_t sssp16_dispatch(ear_plan_s *p, OutT *out, int64_t ldo, int32_t L, int32_t row0, int32_t rows,
                                    const int32_t *trows, int cap, int smem, int32_t *ws,
                                    unsigned long long *d_stats, cudaStream_t st) {
  switch (p->r_k16) {
    case 4: return sssp16_launch<NTS, 4, DistT, OutT>(p, out, ldo, L, row0, rows, trows, cap, smem, ws, d_stats, st);
    case 8: return sssp16_launch<NTS, 8, DistT, OutT>(p, out, ldo, L, row0, rows, trows, cap, smem, ws, d_stats, st);
    case 12: return sssp16_launch<NTS, 12, DistT, OutT>(p, out, ldo, L, row0, rows, trows, cap, smem, ws, d_stats, st);
    default: return sssp16_launch<NTS, 16, DistT, OutT>(p, out, ldo, L, row0, rows, trows, cap, smem, ws, d_stats, st);
  }
}

// rows [row0, row0 + rows) (or the tile rows listed in trows) into out (u16 or int32, ldo), row length L
// (a multiple of 8, >= N_r); *applied = false when the route does not apply or a distance saturated
template <typename OutT>
static ear_status_t sssp16_rows(ear_plan_s *p, OutT *out, int64_t ldo, int32_t L, int32_t row0, int32_t rows,
                                const int32_t *trows, bool *applied, cudaStream_t st) {
  *applied = false;
  EAR_TRY(ell16_prepare(p, st));
  if (p->r_k16 <= 0 || L % 8 != 0 || L < p->n_reduced || L >= 0xFFFF) return EAR_OK;
  int dev = 0, max_smem = 0;
  EAR_CUDA_TRY(cudaGetDevice(&dev));
  EAR_CUDA_TRY(cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  int per_sm_smem = 0;
  EAR_CUDA_TRY(cudaDeviceGetAttribute(&per_sm_smem, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev));
  // list capacity: as large as lets the most sources share an SM (a near-far frontier of the paper's
  // sparse reduced graphs stays well below 1k), never below 256; 1 KB per CTA is the driver's, 256 B
  // the kernel's static shared memory
  auto fit = [&](int db, int *cap_out) {
    for (int per = SSSP16_MAX_CTAS; per >= 1; --per) {
      const int budget = std::min(max_smem, per_sm_smem / per - 1024 - 256);
      const int c = ((budget - sssp16_smem(L, 0, db)) / 4) & ~7;
      if (c >= 256) {
        *cap_out = std::min(c, 4096);
        return per;
      }
    }
    return 0;
  };
  // the row as u32 (one ATOMS.MIN per relaxation) when four sources still share an SM, else the row
  // type that fits more of them (u16: 16-bit CAS relaxations, half the bytes) -- measured, cfg2 u32 4.8
  // vs 5.9 ms, cfg3_f60 u16 29.7 vs 31.7 ms, cfg4 u16 136 vs 199 ms
  int cap4 = 0, cap2 = 0;
  const int per4 = fit(4, &cap4), per2 = fit(2, &cap2);
  int db = per4 >= 4 || per4 >= per2 ? 4 : 2;
  if (const char *e = getenv("EAR_SSSP16_DIST")) db = atoi(e) == 2 ? 2 : atoi(e) == 4 && per4 > 0 ? 4 : db;   // lab
  int cap = db == 4 ? cap4 : cap2;
  if (cap == 0) return EAR_OK;
  if (const char *e = getenv("EAR_SSSP16_CAP")) cap = std::max(16, std::min(cap, atoi(e) & ~7));   // test knob: overflow
  const int smem = sssp16_smem(L, cap, db);
  if (rows <= 0) { *applied = true; return EAR_OK; }
  int32_t *ws = nullptr;   // counter, saturation flag, watermark, -, one done flag per row
  const size_t wsb = sizeof(int32_t) * (4 + (size_t)rows);
  EAR_CUDA_TRY(cudaMallocAsync((void **)&ws, wsb, st));
  EAR_CUDA_TRY(dev_memset(ws, 0, wsb, st));
  static unsigned long long *d_stats = nullptr;
  static const bool want_stats = getenv("EAR_SSSP_STATS") != nullptr;
  if (want_stats && !d_stats) EAR_CUDA_TRY(cudaMalloc((void **)&d_stats, 16));
  if (want_stats) EAR_CUDA_TRY(dev_memset(d_stats, 0, 16, st));
  unsigned long long *stt = want_stats ? d_stats : nullptr;
  ear_status_t s = EAR_OK;
  static const int nt_lab = [] {
    const char *e = getenv("EAR_SSSP16_NT");   // lab knob: 128 threads per source
    return e ? atoi(e) : 0;
  }();
  if (nt_lab == 128) {
    s = db == 4 ? sssp16_dispatch<128, uint32_t>(p, out, ldo, L, row0, rows, trows, cap, smem, ws, stt, st)
                : sssp16_dispatch<128, uint16_t>(p, out, ldo, L, row0, rows, trows, cap, smem, ws, stt, st);
  } else if (db == 4) {
    s = sssp16_dispatch<SSSP16_NT, uint32_t>(p, out, ldo, L, row0, rows, trows, cap, smem, ws, stt, st);
  } else {
    s = sssp16_dispatch<SSSP16_NT, uint16_t>(p, out, ldo, L, row0, rows, trows, cap, smem, ws, stt, st);
  }
  int32_t h_sat = 1;
  if (s == EAR_OK) {
    Readback rb(st);
    cudaError_t e = rb.get(&h_sat, ws + 1, 4);
    if (e == cudaSuccess) e = rb.sync();
    if (e != cudaSuccess) { set_error("sssp16: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  }
  cudaFreeAsync(ws, st);
  if (s == EAR_OK) *applied = h_sat == 0;
  return s;
}

ear_status_t sssp_rows16(ear_plan_s *p, uint16_t *D16, int64_t ld16, bool *applied, cudaStream_t st) {
  NvtxRange nvtx_("ear: Phase II by per-source SSSP");
  const int32_t L = (int32_t)round_up(std::max(p->n_reduced, 1), 8);
  if (ld16 < L) { *applied = false; return EAR_OK; }
  return sssp16_rows<uint16_t>(p, D16, ld16, L, 0, p->n_reduced, nullptr, applied, st);
}

// Rows [row0, row0 + rows) of D (row-major, ldd) by per-source Bellman-Ford on G^r.
ear_status_t sssp_rows(ear_plan_s *p, int32_t *D, int64_t ldd, int32_t Np, int32_t row0, int32_t rows,
                       const int32_t *trows,
                       cudaStream_t st) {
  EAR_TRY(sssp_prepare(p, st));
  if (rows <= 0) return EAR_OK;
  static const bool u16_off = [] {
    const char *e = getenv("EAR_SSSP16");   // 0: the int32 kernels (A/B)
    return e && atoi(e) == 0;
  }();
  if (!u16_off && rows > 1) {   // (one row: the packed FW's precheck -- latency, not throughput)
    bool applied = false;
    EAR_TRY(sssp16_rows<int32_t>(p, D, ldd, Np, row0, rows, trows, &applied, st));
    if (applied) return EAR_OK;
  }
  const int W = (Np + 31) / 32;
  static unsigned long long *d_stats = nullptr;
  static const bool want_stats = getenv("EAR_SSSP_STATS") != nullptr;
  if (want_stats && !d_stats) EAR_CUDA_TRY(cudaMalloc((void **)&d_stats, 32));
  if (want_stats) EAR_CUDA_TRY(dev_memset(d_stats, 0, 32, st));
  int dev = 0, nsm = 148;
  EAR_CUDA_TRY(cudaGetDevice(&dev));
  EAR_CUDA_TRY(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  int max_smem = 0;
  EAR_CUDA_TRY(cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  const int smem_s = 4 * Np + 4 * SSSP_LIST + 8 * W;
  if (smem_s + 64 <= max_smem) {
    // distance row on chip; adjacency as ELL rows of K arcs when the max degree allows (else CSR)
    if (!p->r_arcs) {
      int32_t *d_md = nullptr, md = 0;
      EAR_CUDA_TRY(cudaMallocAsync((void **)&d_md, 4, st));
      EAR_CUDA_TRY(dev_memset(d_md, 0, 4, st));
      EAR_LAUNCH(k_max_deg, (int)std::min<int64_t>(ceil_div(p->n_reduced, 256), 4096), 256, 0, st)(
          p->r_rowptr, p->n_reduced, d_md);
      {
        Readback rb(st);
        EAR_CUDA_TRY(rb.get(&md, d_md, 4));
        EAR_CUDA_TRY(rb.sync());
      }
      cudaFreeAsync(d_md, st);
      p->r_ell_k = md <= 4 ? 4 : md <= 8 ? 8 : md <= 12 ? 12 : md <= 16 ? 16 : 0;
      if (p->r_ell_k > 0) {
        EAR_CUDA_TRY(cudaMallocAsync((void **)&p->r_arcs, sizeof(int2) * (size_t)p->r_ell_k * std::max(p->n_reduced, 1), st));
        EAR_LAUNCH(k_build_ell, (int)std::min<int64_t>(ceil_div(p->n_reduced, 256), 4096), 256, 0, st)(
            p->r_rowptr, p->r_col, p->r_w, p->n_reduced, p->r_ell_k, reinterpret_cast<int2 *>(p->r_arcs));
      } else {
        EAR_CUDA_TRY(cudaMallocAsync((void **)&p->r_arcs, sizeof(int2) * (size_t)std::max(p->n_rarcs, 1), st));
        if (p->n_rarcs > 0)
          EAR_LAUNCH(k_pack_arcs, (int)std::min<int64_t>(ceil_div(p->n_rarcs, 256), 4096), 256, 0, st)(
              p->r_col, p->r_w, p->n_rarcs, reinterpret_cast<int2 *>(p->r_arcs));
      }
    }
    constexpr int NTS = 512;
    // list-driven rounds win when two or more sources share an SM (cfg2: 6.7 vs 10.7 ms); with one
    // resident source per SM the bitmap-scan rounds are faster (cfg4: 475 vs 533 ms)
    const int list_smem = 4 * Np + 8 * std::min(Np, (max_smem - (4 * Np + 8 * W + 64)) / 8) + 8 * W;
    if (2 * list_smem + 2048 <= max_smem + 1024) {
      switch (p->r_ell_k) {
        case 4: return sssp_list_launch<NTS, 4>(p, D, ldd, Np, row0, rows, trows, max_smem, nsm, want_stats ? d_stats : nullptr, st);
        case 8: return sssp_list_launch<NTS, 8>(p, D, ldd, Np, row0, rows, trows, max_smem, nsm, want_stats ? d_stats : nullptr, st);
        case 12: return sssp_list_launch<NTS, 12>(p, D, ldd, Np, row0, rows, trows, max_smem, nsm, want_stats ? d_stats : nullptr, st);
        case 16: return sssp_list_launch<NTS, 16>(p, D, ldd, Np, row0, rows, trows, max_smem, nsm, want_stats ? d_stats : nullptr, st);
        default: break;
      }
    }
    switch (p->r_ell_k) {
      case 4: return sssp_launch<NTS, 4>(p, D, ldd, Np, row0, rows, trows, smem_s, nsm, want_stats ? d_stats : nullptr, st);
      case 8: return sssp_launch<NTS, 8>(p, D, ldd, Np, row0, rows, trows, smem_s, nsm, want_stats ? d_stats : nullptr, st);
      case 12: return sssp_launch<NTS, 12>(p, D, ldd, Np, row0, rows, trows, smem_s, nsm, want_stats ? d_stats : nullptr, st);
      case 16: return sssp_launch<NTS, 16>(p, D, ldd, Np, row0, rows, trows, smem_s, nsm, want_stats ? d_stats : nullptr, st);
      default: return sssp_launch<NTS, 0>(p, D, ldd, Np, row0, rows, trows, smem_s, nsm, want_stats ? d_stats : nullptr, st);
    }
  }
  const int smem = 2 * W * 4;
  EAR_CUDA_TRY(smem_attr((const void *)k_sssp_bf, smem));
  int per_sm = 1;
  EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_sssp_bf, NT, smem));
  // concurrent rows live in L2: cap the number of resident sources (rows of 4*Np bytes) near 96 MB
  const int64_t l2_rows = std::max<int64_t>(nsm, (96ll << 20) / (4ll * Np));
  const int64_t grid = std::min<int64_t>({(int64_t)rows, (int64_t)nsm * std::max(per_sm, 1), l2_rows});
  int s = prof_begin(PK_SSSP, st);
  EAR_LAUNCH(k_sssp_bf, (unsigned)grid, NT, smem, st)(p->r_rowptr, p->r_col, p->r_w, p->n_reduced, Np, D, ldd, row0,
                                                      rows, trows, want_stats ? d_stats : nullptr);
  if (want_stats) {
    unsigned long long h[4];
    EAR_CUDA_TRY(cudaMemcpyAsync(h, d_stats, 32, cudaMemcpyDeviceToHost, st));
    EAR_CUDA_TRY(cudaStreamSynchronize(st));
    fprintf(stderr, "[sssp] grid=%lld rows=%d rounds=%llu (%.1f/source) relax=%llu (%.0f/source) improve=%llu visits=%llu arcs=%d\n",
            (long long)grid, rows, h[0], (double)h[0] / rows, h[1], (double)h[1] / rows, h[2], h[3], p->n_rarcs);
  }
  prof_end(s, st, (double)rows * (double)p->n_rarcs);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

}  // namespace ear
