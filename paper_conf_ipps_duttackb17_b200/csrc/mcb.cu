// Minimum cycle basis (paper sec. 3) of G, computed on its reduced graph
// G^r (Lemma 3.1: W(MCB(G)) = W(MCB(G^r)), same dimension) by de Pina's Algorithm 2
// with the paper's processing phase (sec. 3.3.2):
//
//   pre-processing   Phase I (ear_decompose): G^r = terminals + one edge per maximal degree-two chain
//                    (closed ears are self-loops, parallel chains parallel edges) + the direct
//                    terminal-terminal edges of G.
//   trees            one shortest-path tree T_z per vertex z of G^r ("single source shortest path trees
//                    from each node in the reduced graph"), read off the reduced APSP matrix D of
//                    Phase II (the blocked FW): the parent of u is a tight edge (D[z][v] + w = D[z][u]).
//                    Ties are broken by a 40-bit hash perturbation of the edge weights compared
//                    lexicographically after the weight -- the shortest paths it selects are unique with
//                    high probability, hence consistent, which the candidate set below assumes -- a
//                    Bellman-Ford pass over the tight arcs (reading M3 of DESIGN.md).
//   candidates       the Mehlhorn-Michail set A: for every tree T_z and non-tree edge
//                    e = uv whose tree paths meet only at z (LCA(u,v) = z), the cycle C_ze of weight
//                    d_z(u) + W(uv) + d_z(v); sorted by weight once.
//   phases           f = m - n + k phases; phase i: the labels l_z(u) = <path_z(u), S_i> of Algorithm 3
//                    (one warp per tree, level by level from the root); the first candidate in
//                    weight order with l_z(u) xor l_z(v) xor S_i(e) = 1 (persistent CTAs over
//                    batches with an early exit, no host round trip); C_i's incidence vector on E'
//                    (walk of its two tree paths); the independence test S_j ^= S_i for every later
//                    witness with <C_i, S_j> = 1 (lines 4-8; one warp per witness).
//   post-processing  a basis cycle is expanded into G's vertices on request (sec. 3.3.3, P:376-379:
//                    every chain edge e_P replaced by its chain P).
// The witness coordinates are the non-tree edges E' of a fixed spanning forest T of G^r: the shortest-
// path tree of each component's smallest vertex ("T any spanning tree").
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdio>
#include <vector>

#include "common.cuh"

struct ear_mcb_s {
  ear_plan_s *plan = nullptr;   // owned: descriptors, chain segments (post-processing)
  cudaStream_t st = nullptr;
  int32_t n = 0, N = 0, f = 0, k = 0, Np = 0, dmax = 0;
  int64_t M = 0, ncand = 0, weight = 0;
  int32_t *eu = nullptr, *ev = nullptr, *ew = nullptr, *ech = nullptr;   // G^r edges [M]
  int32_t *PE = nullptr;                                                 // [N x N] parent edge in T_z
  int32_t *cyc_z = nullptr, *cyc_e = nullptr;                            // basis cycle i = C_{z e}
  int64_t *cyc_w = nullptr;
  int32_t *tid2v = nullptr;                                              // [N] caller id of each tid
};

namespace ear {
namespace {

constexpr int NT = 256;
constexpr int64_t H_INF = INT64_MAX;
constexpr int BATCH = 1 << 16;   // candidates per scan work item

int grid_for(int64_t n) { return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, NT), 148 * 16)); }

__device__ __forceinline__ int64_t hperturb(int32_t e) {   // 40-bit splitmix64 hash of the edge id
  uint64_t x = (uint64_t)(uint32_t)e + 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  x ^= x >> 31;
  return (int64_t)(x >> 24);
}
__device__ __forceinline__ int32_t other_end(const int32_t *eu, const int32_t *ev, int32_t e, int32_t x) {
  return eu[e] == x ? ev[e] : eu[e];
}
__device__ __forceinline__ uint32_t bit(const uint32_t *v, int32_t i) { return (v[i >> 5] >> (i & 31)) & 1u; }

// ---- G^r edges: one per chain segment (its ends and length from any of its vertices), then the direct
// terminal-terminal edges (reduced arcs without an interior vertex, taken from their smaller end)
__global__ void k_chain_edges(int32_t nch, const int32_t *seg_start, const int32_t *seg_vert, const VDesc *desc,
                              int32_t *eu, int32_t *ev, int32_t *ew, int32_t *ech) {
  for (int32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < nch; c += gridDim.x * blockDim.x) {
    const VDesc d = desc[seg_vert[seg_start[c]]];
    eu[c] = d.p; ev[c] = d.q; ew[c] = d.cp + d.cq; ech[c] = c;
  }
}
__global__ void k_direct_flag(int64_t A, const int32_t *ru, const int32_t *rv, const int32_t *rx, int32_t *flag) {
  for (int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; a < A; a += (int64_t)gridDim.x * blockDim.x)
    flag[a] = rx[a] < 0 && ru[a] < rv[a];
}
__global__ void k_direct_edges(int64_t A, const int32_t *ru, const int32_t *rv, const int32_t *rw, const int32_t *flag,
                               const int32_t *pos, int32_t base, int32_t *eu, int32_t *ev, int32_t *ew, int32_t *ech) {
  for (int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; a < A; a += (int64_t)gridDim.x * blockDim.x)
    if (flag[a]) {
      const int32_t e = base + pos[a];
      eu[e] = ru[a]; ev[e] = rv[a]; ew[e] = rw[a]; ech[e] = -1;
    }
}
__global__ void k_edge_keys(int32_t k, const int32_t *eu, const int32_t *ev, const int32_t *ew, uint64_t *key,
                            int32_t *w) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < k; i += gridDim.x * blockDim.x) {
    key[i] = ((uint64_t)(uint32_t)eu[i] << 32) | (uint32_t)ev[i];
    w[i] = ew[i];
  }
}
__global__ void k_edge_unkey(int32_t k, const uint64_t *key, const int32_t *w, int32_t *eu, int32_t *ev, int32_t *ew) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < k; i += gridDim.x * blockDim.x) {
    eu[i] = (int32_t)(key[i] >> 32);
    ev[i] = (int32_t)(key[i] & 0xFFFFFFFFu);
    ew[i] = w[i];
  }
}
// CSR of G^r (both arc directions; a self-loop gives two arcs at its vertex, never tight)
__global__ void k_deg(int64_t M, const int32_t *eu, const int32_t *ev, int32_t *deg) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < M; e += (int64_t)gridDim.x * blockDim.x) {
    atomicAdd(&deg[eu[e]], 1);
    atomicAdd(&deg[ev[e]], 1);
  }
}
__global__ void k_arcs(int64_t M, const int32_t *eu, const int32_t *ev, int32_t *cur, int32_t *arc_v, int32_t *arc_e) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < M; e += (int64_t)gridDim.x * blockDim.x) {
    int32_t p = atomicAdd(&cur[eu[e]], 1);
    arc_v[p] = ev[e]; arc_e[p] = (int32_t)e;
    p = atomicAdd(&cur[ev[e]], 1);
    arc_v[p] = eu[e]; arc_e[p] = (int32_t)e;
  }
}

// ---- shortest-path trees T_z from D, ties broken by (H, edge id): H_z(u) = min over tight arcs (v -> u)
// of H_z(v) + h(e); iterated to the fixed point (Bellman-Ford over the tight arcs, hop-depth rounds)
__global__ void k_tree_init(int32_t N, int64_t *H, int32_t *PE) {
  const int64_t NN = (int64_t)N * N;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < NN; i += (int64_t)gridDim.x * blockDim.x) {
    H[i] = (i / N == i % N) ? 0 : H_INF;
    PE[i] = -1;
  }
}
__global__ void k_tree_round(int32_t N, int32_t Np, const int32_t *__restrict__ D, const int32_t *__restrict__ rowptr,
                             const int32_t *__restrict__ arc_v, const int32_t *__restrict__ arc_e,
                             const int32_t *__restrict__ ew, int64_t *H, int32_t *PE, int32_t *changed) {
  const int64_t NN = (int64_t)N * N;
  int any = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < NN; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t z = (int32_t)(i / N), u = (int32_t)(i % N);
    const int32_t *Dz = D + (int64_t)z * Np;
    const int32_t du = Dz[u];
    if (u == z || du >= INF) continue;
    int64_t best = H[i];
    int32_t bpe = PE[i];
    for (int32_t a = rowptr[u]; a < rowptr[u + 1]; ++a) {
      const int32_t v = arc_v[a], e = arc_e[a];
      if (v == u) continue;
      if (Dz[v] >= INF || Dz[v] + ew[e] != du) continue;
      const int64_t hv = H[(int64_t)z * N + v];
      if (hv == H_INF) continue;
      const int64_t c = hv + hperturb(e);
      if (c < best || (c == best && e < bpe)) { best = c; bpe = e; }
    }
    if (bpe != PE[i] || best != H[i]) {
      H[i] = best;
      PE[i] = bpe;
      any = 1;
    }
  }
  if (__syncthreads_or(any) && threadIdx.x == 0) *changed = 1;
}
// hop depth and branch (the child of z on the path z -> u) of every (z, u); -1 for unreachable
__global__ void k_depth_branch(int32_t N, const int32_t *eu, const int32_t *ev, const int32_t *PE, int32_t *depth,
                               int32_t *BR, int32_t *dmax) {
  const int64_t NN = (int64_t)N * N;
  int32_t mx = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < NN; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t z = (int32_t)(i / N), u = (int32_t)(i % N);
    const int32_t *P = PE + (int64_t)z * N;
    if (u == z) { depth[i] = 0; BR[i] = z; continue; }
    if (P[u] < 0) { depth[i] = -1; BR[i] = -1; continue; }
    int32_t x = u, d = 0, br = u;
    while (x != z) {
      const int32_t p = other_end(eu, ev, P[x], x);
      if (p == z) br = x;
      x = p;
      ++d;
    }
    depth[i] = d;
    BR[i] = br;
    mx = max(mx, d);
  }
  mx = __reduce_max_sync(0xFFFFFFFFu, mx);
  if ((threadIdx.x & 31) == 0) atomicMax(dmax, mx);
}
// level order of every tree: counts per (tree, depth), per-tree exclusive scan, scatter
__global__ void k_level_count(int32_t N, int32_t L, const int32_t *depth, int32_t *cnt) {
  const int64_t NN = (int64_t)N * N;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < NN; i += (int64_t)gridDim.x * blockDim.x)
    if (depth[i] >= 0) atomicAdd(&cnt[(i / N) * L + depth[i]], 1);
}
__global__ void k_level_scan(int32_t N, int32_t L, int32_t *cnt, int32_t *start) {   // one thread per tree
  for (int32_t z = blockIdx.x * blockDim.x + threadIdx.x; z < N; z += gridDim.x * blockDim.x) {
    int32_t s = 0;
    for (int32_t d = 0; d < L; ++d) {
      start[(int64_t)z * (L + 1) + d] = s;
      s += cnt[(int64_t)z * L + d];
      cnt[(int64_t)z * L + d] = 0;   // reused as the scatter cursor
    }
    start[(int64_t)z * (L + 1) + L] = s;
  }
}
__global__ void k_level_scatter(int32_t N, int32_t L, const int32_t *depth, const int32_t *start, int32_t *cur,
                                int32_t *order) {
  const int64_t NN = (int64_t)N * N;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < NN; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t d = depth[i];
    if (d < 0) continue;
    const int64_t z = i / N;
    const int32_t p = start[z * (L + 1) + d] + atomicAdd(&cur[z * L + d], 1);
    order[z * N + p] = (int32_t)(i % N);
  }
}
// the level order with what a label step needs per node: {u, parent, coordinate of the parent edge
// (-1 for tree edges of T), 0} -- one 16-byte load per node in k_labels
__global__ void k_order4(int32_t N, int32_t L, const int32_t *order, const int32_t *lstart, const int32_t *PE,
                         const int32_t *eu, const int32_t *ev, const int32_t *coord, int4 *ord4) {
  const int64_t NN = (int64_t)N * N;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < NN; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t z = i / N;
    const int32_t idx = (int32_t)(i % N);
    if (idx < lstart[z * (L + 1) + 1] || idx >= lstart[z * (L + 1) + L]) continue;   // the root, unreachable
    const int32_t u = order[i], pe = PE[z * N + u];
    ord4[i] = make_int4(u, other_end(eu, ev, pe, u), coord[pe], 0);
  }
}

// the fixed spanning forest T: the tree of each component's smallest vertex; E' coordinates
__global__ void k_mark_tree(int32_t N, const int32_t *lab, const int32_t *PE, int32_t *intree, int32_t *roots) {
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < N; u += gridDim.x * blockDim.x) {
    const int32_t r = lab[u];
    if (r == u) atomicAdd(roots, 1);
    else intree[PE[(int64_t)r * N + u]] = 1;
  }
}
__global__ void k_not(int64_t M, const int32_t *intree, int32_t *flag) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < M; e += (int64_t)gridDim.x * blockDim.x)
    flag[e] = !intree[e];
}
__global__ void k_coord(int64_t M, const int32_t *intree, const int32_t *pos, int32_t *coord) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < M; e += (int64_t)gridDim.x * blockDim.x)
    coord[e] = intree[e] ? -1 : pos[e];
}

// ---- the candidate set A: (z, e) with LCA_z(u, v) = z and e not a tree edge of T_z; key = weight << 32 |
// the top 32 bits of the perturbation (weight order, ties by the tree system's unique order)
__global__ void k_candidates(int32_t N, int64_t M, int32_t Np, const int32_t *__restrict__ D,
                             const int32_t *__restrict__ eu, const int32_t *__restrict__ ev,
                             const int32_t *__restrict__ ew, const int32_t *__restrict__ PE,
                             const int32_t *__restrict__ BR, const int64_t *__restrict__ H,
                             unsigned long long *count, uint64_t *keys, int64_t *vals) {
  const int64_t tot = (int64_t)N * M;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < tot; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t z = (int32_t)(i / M), e = (int32_t)(i % M);
    const int32_t u = eu[e], v = ev[e];
    int64_t W, Hk;
    if (u == v) {   // a self-loop (closed ear) is a cycle by itself, generated at its vertex
      if (u != z) continue;
      W = ew[e];
      Hk = hperturb(e);
    } else {
      const int32_t *Dz = D + (int64_t)z * Np;
      if (Dz[u] >= INF || Dz[v] >= INF) continue;
      const int64_t zN = (int64_t)z * N;
      if (PE[zN + u] == e || PE[zN + v] == e) continue;
      if (!(u == z || v == z || BR[zN + u] != BR[zN + v])) continue;
      W = (int64_t)Dz[u] + ew[e] + Dz[v];
      Hk = H[zN + u] + hperturb(e) + H[zN + v];
    }
    const unsigned long long k = atomicAdd(count, 1ull);
    if (keys) {
      keys[k] = ((uint64_t)W << 32) | (uint64_t)((uint64_t)Hk >> 31);
      vals[k] = ((int64_t)z << 32) | (uint32_t)e;
    }
  }
}

__global__ void k_witness_init(int32_t f, int32_t Wd, uint32_t *S) {
  const int64_t tot = (int64_t)f * Wd;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < tot; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / Wd), w = (int32_t)(i % Wd);
    S[i] = (r >> 5) == w ? (1u << (r & 31)) : 0u;
  }
}

// ---- phase i, 1: labels l_z(u) = l_z(parent) xor S_i(parent edge) (0 for tree edges of T, which have
// no coordinate), Algorithm 3; one WARP per tree, level by level (a warp barrier per level), the labels
// as bits in shared memory (N bits per tree), then copied to Lbits[z]
constexpr int LW = 8;   // trees (warps) per CTA
__global__ void __launch_bounds__(LW * 32) k_labels(int32_t N, int32_t L, const int4 *__restrict__ ord4,
                                                    const int32_t *__restrict__ start, const uint32_t *__restrict__ Si,
                                                    uint32_t *__restrict__ Lbits, int32_t Wn) {
  extern __shared__ uint32_t lbits[];   // [LW][Wn]
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  const int32_t z = blockIdx.x * LW + wi;
  if (z >= N) return;
  uint32_t *lab = lbits + wi * Wn;
  const int4 *ord = ord4 + (int64_t)z * N;
  const int32_t *st = start + (int64_t)z * (L + 1);
  for (int32_t w = lane; w < Wn; w += 32) lab[w] = 0;
  __syncwarp();
  for (int32_t d = 1; d < L; ++d) {
    const int32_t b = st[d], e = st[d + 1];
    if (b == e) break;
    for (int32_t idx = b + lane; idx < e; idx += 32) {
      const int4 r = ord[idx];   // {u, parent, coordinate of the parent edge or -1}
      if (bit(lab, r.y) ^ (r.z >= 0 ? bit(Si, r.z) : 0u)) atomicOr(&lab[r.x >> 5], 1u << (r.x & 31));
    }
    __syncwarp();
  }
  for (int32_t w = lane; w < Wn; w += 32) Lbits[(int64_t)z * Wn + w] = lab[w];
}

struct PhaseState {
  unsigned long long best;   // first candidate index with odd parity
  int32_t next_batch;
  int32_t missing;           // a phase found no candidate (cannot happen: a fundamental cycle is odd)
  long long weight;
};

// ---- phase i, 2: the first candidate in weight order non-orthogonal to S_i (persistent CTAs take batches
// in order and stop once a batch lies beyond the best index found)
__global__ void __launch_bounds__(NT) k_scan(int64_t ncand, const int64_t *__restrict__ vals,
                                             const int32_t *__restrict__ eu, const int32_t *__restrict__ ev,
                                             const int32_t *__restrict__ coord, const uint32_t *__restrict__ Si,
                                             const uint32_t *__restrict__ Lbits, int32_t Wn, PhaseState *ps) {
  __shared__ int32_t bsh;
  for (;;) {
    if (threadIdx.x == 0) bsh = atomicAdd(&ps->next_batch, 1);
    __syncthreads();
    const int64_t b0 = (int64_t)bsh * BATCH;
    __syncthreads();
    if (b0 >= ncand || (unsigned long long)b0 > *(volatile unsigned long long *)&ps->best) return;
    const int64_t b1 = min(ncand, b0 + BATCH);
    for (int64_t c = b0 + threadIdx.x; c < b1; c += blockDim.x) {
      const int64_t zv = vals[c];
      const int32_t z = (int32_t)(zv >> 32), e = (int32_t)(uint32_t)zv;
      const int32_t u = eu[e], v = ev[e], k = coord[e];
      const uint32_t *Lz = Lbits + (int64_t)z * Wn;
      const uint32_t par = bit(Lz, u) ^ bit(Lz, v) ^ (k >= 0 ? bit(Si, k) : 0u);
      if (par) {
        atomicMin(&ps->best, (unsigned long long)c);
        break;   // later candidates of this thread cannot be first
      }
    }
  }
}

// ---- phase i, 3: record C_i and its incidence vector on E' (the xor of its two tree paths and e)
__global__ void k_cycle(int32_t i, const uint64_t *__restrict__ keys, const int64_t *__restrict__ vals,
                        const int32_t *__restrict__ eu, const int32_t *__restrict__ ev, const int32_t *__restrict__ PE,
                        const int32_t *__restrict__ coord, int32_t N, uint32_t *C, int32_t Wd, PhaseState *ps,
                        int32_t *cyc_z, int32_t *cyc_e, int64_t *cyc_w) {
  for (int32_t w = threadIdx.x; w < Wd; w += blockDim.x) C[w] = 0;
  __syncthreads();
  const unsigned long long best = ps->best;
  if (best == ~0ull) {
    if (threadIdx.x == 0) { ps->missing = 1; cyc_z[i] = -1; cyc_e[i] = -1; cyc_w[i] = 0; }
    return;
  }
  const int32_t z = (int32_t)(vals[best] >> 32), e = (int32_t)(uint32_t)vals[best];
  const int32_t *P = PE + (int64_t)z * N;
  if (threadIdx.x == 0) {
    const int64_t W = (int64_t)(keys[best] >> 32);
    cyc_z[i] = z; cyc_e[i] = e; cyc_w[i] = W;
    ps->weight += W;
    if (coord[e] >= 0) atomicXor(&C[coord[e] >> 5], 1u << (coord[e] & 31));
  }
  if (threadIdx.x < 2 && eu[e] != ev[e]) {
    for (int32_t x = threadIdx.x == 0 ? eu[e] : ev[e]; x != z;) {
      const int32_t pe = P[x], k = coord[pe];
      if (k >= 0) atomicXor(&C[k >> 5], 1u << (k & 31));
      x = other_end(eu, ev, pe, x);
    }
  }
}

// ---- phase i, 4: independence test, S_j ^= S_i for every j > i with <C_i, S_j> = 1; one warp per witness;
// then the scan state is reset for the next phase
__global__ void k_update(int32_t i, int32_t f, int32_t Wd, uint32_t *S, const uint32_t *C, PhaseState *ps) {
  const int32_t lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const uint32_t *Si = S + (int64_t)i * Wd;
  for (int64_t j = i + 1 + warp; j < f; j += nw) {
    uint32_t *Sj = S + j * Wd;
    uint32_t p = 0;
    for (int32_t w = lane; w < Wd; w += 32) p ^= __popc(Sj[w] & C[w]) & 1u;
    p = __reduce_xor_sync(0xFFFFFFFFu, p);
    if (p)
      for (int32_t w = lane; w < Wd; w += 32) Sj[w] ^= Si[w];
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    ps->best = ~0ull;
    ps->next_batch = 0;
  }
}

__global__ void k_ps_init(PhaseState *ps) {
  ps->best = ~0ull;
  ps->next_batch = 0;
  ps->missing = 0;
  ps->weight = 0;
}

__global__ void k_tid2v(int32_t n, const int32_t *tid, int32_t *tid2v) {
  for (int32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x)
    if (tid[v] >= 0) tid2v[tid[v]] = v;
}

// ---- post-processing (sec. 3.3.3): basis cycle i as a closed sequence of G's vertices (caller ids), the
// start vertex not repeated: z -> ... -> u (tree path), e, v -> ... -> z (tree path); every chain edge is
// replaced by its chain's vertices (segments are sorted by the distance from their left end eu)
__device__ void emit_edge(int32_t e, int32_t from, const int32_t *eu, const int32_t *ech, const int32_t *seg_start,
                          const int32_t *seg_vert, const int32_t *tid2v, int32_t *out, int32_t cap, int32_t *len) {
  if (*len < cap && out) out[*len] = tid2v[from];
  ++*len;
  const int32_t c = ech[e];
  if (c < 0) return;
  const int32_t b = seg_start[c], t = seg_start[c + 1];
  const bool fwd = eu[e] == from;
  for (int32_t k = 0; k < t - b; ++k) {
    if (*len < cap && out) out[*len] = seg_vert[fwd ? b + k : t - 1 - k];
    ++*len;
  }
}
__global__ void k_expand_cycle(int32_t i, int32_t N, const int32_t *cyc_z, const int32_t *cyc_e, const int32_t *eu,
                               const int32_t *ev, const int32_t *ech, const int32_t *PE, const int32_t *seg_start,
                               const int32_t *seg_vert, const int32_t *tid2v, int32_t *out, int32_t cap,
                               int32_t *len_out, int32_t *scratch) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  const int32_t z = cyc_z[i], e = cyc_e[i], u = eu[e], v = ev[e];
  const int32_t *P = PE + (int64_t)z * N;
  int32_t len = 0;
  if (u == v) {
    emit_edge(e, u, eu, ech, seg_start, seg_vert, tid2v, out, cap, &len);
    *len_out = len;
    return;
  }
  // tree path z -> u: collect u's ancestors' edges (scratch), then emit them from the root down
  int32_t np = 0;
  for (int32_t x = u; x != z; x = other_end(eu, ev, P[x], x)) scratch[np++] = P[x];
  int32_t at = z;
  for (int32_t k = np - 1; k >= 0; --k) {
    emit_edge(scratch[k], at, eu, ech, seg_start, seg_vert, tid2v, out, cap, &len);
    at = other_end(eu, ev, scratch[k], at);
  }
  emit_edge(e, u, eu, ech, seg_start, seg_vert, tid2v, out, cap, &len);
  for (int32_t x = v; x != z; x = other_end(eu, ev, P[x], x)) emit_edge(P[x], x, eu, ech, seg_start, seg_vert, tid2v,
                                                                        out, cap, &len);
  *len_out = len;
}

struct Scratch {
  cudaStream_t st;
  std::vector<void *> ptrs;
  template <class T>
  ear_status_t get(T **p, int64_t n) {
    if (cudaMallocAsync((void **)p, sizeof(T) * (size_t)std::max<int64_t>(n, 1), st) != cudaSuccess) {
      cudaGetLastError();
      set_error("ear_mcb: out of device memory (%lld bytes)", (long long)(sizeof(T) * n));
      return EAR_ENOMEM;
    }
    ptrs.push_back(*p);
    return EAR_OK;
  }
  ~Scratch() {
    for (void *p : ptrs) cudaFreeAsync(p, st);
  }
};

template <class T>
ear_status_t alloc_keep(T **p, int64_t n, cudaStream_t st) {
  if (cudaMallocAsync((void **)p, sizeof(T) * (size_t)std::max<int64_t>(n, 1), st) != cudaSuccess) {
    cudaGetLastError();
    set_error("ear_mcb: out of device memory");
    return EAR_ENOMEM;
  }
  return EAR_OK;
}

ear_status_t exclusive_sum(const int32_t *in, int32_t *out, int64_t n, Scratch &sc) {
  size_t tb = 0;
  EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb, in, out, (int)n, sc.st));
  char *tmp = nullptr;
  EAR_TRY(sc.get(&tmp, (int64_t)tb));
  EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb, in, out, (int)n, sc.st));
  return EAR_OK;
}

template <class T>
ear_status_t read1(T *h, const T *d, cudaStream_t st) {
  Readback rb(st);
  EAR_CUDA_TRY(rb.get(h, d, sizeof(T)));
  EAR_CUDA_TRY(rb.sync());
  return EAR_OK;
}

void mcb_free(ear_mcb_s *m) {
  cudaStream_t st = m->st;
  void *arrs[] = {m->eu, m->ev, m->ew, m->ech, m->PE, m->cyc_z, m->cyc_e, m->cyc_w, m->tid2v};
  for (void *a : arrs)
    if (a) cudaFreeAsync(a, st);
  if (m->plan) {
    cudaStreamSynchronize(st);
    plan_free(m->plan);
    delete m->plan;
  }
}

ear_status_t mcb_build(ear_mcb_s *m, int32_t n, int64_t mm, const int32_t *src, const int32_t *dst, const int32_t *w,
                       cudaStream_t st) {
  m->st = st;
  m->n = n;
  m->plan = new ear_plan_s;
  cudaGetDevice(&m->plan->device);
  EAR_TRY(decompose(n, mm, src, dst, w, 0, st, m->plan));
  ear_plan_s *p = m->plan;
  const int32_t N = m->N = p->n_reduced;
  Scratch sc{st, {}};
  // ---- G^r edge list: chains, then direct edges
  int32_t *dflag = nullptr, *dpos = nullptr;
  EAR_TRY(sc.get(&dflag, p->n_redges));
  EAR_TRY(sc.get(&dpos, p->n_redges));
  int32_t ndirect = 0;
  if (p->n_redges > 0) {
    EAR_LAUNCH(k_direct_flag, grid_for(p->n_redges), NT, 0, st)(p->n_redges, p->re_u, p->re_v, p->re_x, dflag);
    EAR_TRY(exclusive_sum(dflag, dpos, p->n_redges, sc));
    int32_t last_pos = 0, last_flag = 0;
    EAR_TRY(read1(&last_pos, dpos + p->n_redges - 1, st));
    EAR_TRY(read1(&last_flag, dflag + p->n_redges - 1, st));
    ndirect = last_pos + last_flag;
  }
  const int64_t M = m->M = (int64_t)p->n_chains + ndirect;
  EAR_TRY(alloc_keep(&m->eu, M, st));
  EAR_TRY(alloc_keep(&m->ev, M, st));
  EAR_TRY(alloc_keep(&m->ew, M, st));
  EAR_TRY(alloc_keep(&m->ech, M, st));
  if (p->n_chains > 0)
    EAR_LAUNCH(k_chain_edges, grid_for(p->n_chains), NT, 0, st)(p->n_chains, p->seg_start, p->seg_vert, p->desc, m->eu,
                                                                 m->ev, m->ew, m->ech);
  if (ndirect > 0) {
    EAR_LAUNCH(k_direct_edges, grid_for(p->n_redges), NT, 0, st)(p->n_redges, p->re_u, p->re_v, p->re_w, dflag, dpos,
                                                                  p->n_chains, m->eu, m->ev, m->ew, m->ech);
    // Phase I emits the reduced arcs in atomic order: number the direct edges by (u, v) instead, so that
    // edge ids -- hence the perturbation and every tie-break -- are the same on every run
    uint64_t *k0 = nullptr, *k1 = nullptr;
    int32_t *w0 = nullptr, *w1 = nullptr;
    EAR_TRY(sc.get(&k0, ndirect));
    EAR_TRY(sc.get(&k1, ndirect));
    EAR_TRY(sc.get(&w0, ndirect));
    EAR_TRY(sc.get(&w1, ndirect));
    const int32_t c0 = p->n_chains;
    EAR_LAUNCH(k_edge_keys, grid_for(ndirect), NT, 0, st)(ndirect, m->eu + c0, m->ev + c0, m->ew + c0, k0, w0);
    cub::DoubleBuffer<uint64_t> dk(k0, k1);
    cub::DoubleBuffer<int32_t> dw(w0, w1);
    size_t tb = 0;
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dw, ndirect, 0, 64, st));
    char *tmp = nullptr;
    EAR_TRY(sc.get(&tmp, (int64_t)tb));
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dw, ndirect, 0, 64, st));
    EAR_LAUNCH(k_edge_unkey, grid_for(ndirect), NT, 0, st)(ndirect, dk.Current(), dw.Current(), m->eu + c0, m->ev + c0,
                                                           m->ew + c0);
  }
  EAR_TRY(alloc_keep(&m->tid2v, N, st));
  EAR_LAUNCH(k_tid2v, grid_for(n), NT, 0, st)(n, p->tid, m->tid2v);
  // CSR
  int32_t *deg = nullptr, *rowptr = nullptr, *cur = nullptr, *arc_v = nullptr, *arc_e = nullptr;
  EAR_TRY(sc.get(&deg, N + 1));
  EAR_TRY(sc.get(&rowptr, N + 1));
  EAR_TRY(sc.get(&cur, N + 1));
  EAR_TRY(sc.get(&arc_v, 2 * M));
  EAR_TRY(sc.get(&arc_e, 2 * M));
  EAR_CUDA_TRY(dev_memset(deg, 0, sizeof(int32_t) * (N + 1), st));
  if (M > 0) EAR_LAUNCH(k_deg, grid_for(M), NT, 0, st)(M, m->eu, m->ev, deg);
  EAR_TRY(exclusive_sum(deg, rowptr, N + 1, sc));
  EAR_CUDA_TRY(dev_copy(cur, rowptr, sizeof(int32_t) * (N + 1), st));
  if (M > 0) EAR_LAUNCH(k_arcs, grid_for(M), NT, 0, st)(M, m->eu, m->ev, cur, arc_v, arc_e);
  // ---- D = APSP(G^r): Phase II (blocked FW; packed when every distance stays below its cap)
  const int32_t Np = m->Np = (int32_t)round_up(std::max<int64_t>(N, 1), TILE);
  int32_t *D = nullptr;
  EAR_TRY(sc.get(&D, (int64_t)Np * Np));
  EAR_TRY(fw_init_D(p, D, Np, Np, 0, Np, st));
  const int32_t *lab = nullptr;
  EAR_TRY(reduced_labels(p, Np, st, &lab));
  EAR_TRY(fw_single(D, Np, Np, st, lab, N, true, p));
  // ---- trees
  int64_t *H = nullptr;
  int32_t *depth = nullptr, *BR = nullptr, *changed = nullptr;
  EAR_TRY(alloc_keep(&m->PE, (int64_t)N * N, st));
  EAR_TRY(sc.get(&H, (int64_t)N * N));
  EAR_TRY(sc.get(&depth, (int64_t)N * N));
  EAR_TRY(sc.get(&BR, (int64_t)N * N));
  EAR_TRY(sc.get(&changed, 2));
  const int64_t NN = (int64_t)N * N;
  EAR_LAUNCH(k_tree_init, grid_for(NN), NT, 0, st)(N, H, m->PE);
  for (int round = 0; round <= N + 1; ++round) {
    EAR_CUDA_TRY(dev_memset(changed, 0, sizeof(int32_t), st));
    EAR_LAUNCH(k_tree_round, grid_for(NN), NT, 0, st)(N, Np, D, rowptr, arc_v, arc_e, m->ew, H, m->PE, changed);
    int32_t h = 0;
    EAR_TRY(read1(&h, changed, st));
    if (!h) break;
  }
  EAR_CUDA_TRY(dev_memset(changed + 1, 0, sizeof(int32_t), st));
  EAR_LAUNCH(k_depth_branch, grid_for(NN), NT, 0, st)(N, m->eu, m->ev, m->PE, depth, BR, changed + 1);
  EAR_TRY(read1(&m->dmax, changed + 1, st));
  const int32_t L = m->dmax + 1;   // levels 0..dmax
  int32_t *lcnt = nullptr, *lstart = nullptr, *order = nullptr;
  EAR_TRY(sc.get(&lcnt, (int64_t)N * L));
  EAR_TRY(sc.get(&lstart, (int64_t)N * (L + 1)));
  EAR_TRY(sc.get(&order, NN));
  EAR_CUDA_TRY(dev_memset(lcnt, 0, sizeof(int32_t) * (size_t)N * L, st));
  EAR_LAUNCH(k_level_count, grid_for(NN), NT, 0, st)(N, L, depth, lcnt);
  EAR_LAUNCH(k_level_scan, grid_for(N), NT, 0, st)(N, L, lcnt, lstart);
  EAR_LAUNCH(k_level_scatter, grid_for(NN), NT, 0, st)(N, L, depth, lstart, lcnt, order);
  // ---- spanning forest T and the witness coordinates on E'
  int32_t *intree = nullptr, *nflag = nullptr, *npos = nullptr, *coord = nullptr, *roots = nullptr;
  EAR_TRY(sc.get(&intree, M));
  EAR_TRY(sc.get(&nflag, M));
  EAR_TRY(sc.get(&npos, M));
  EAR_TRY(sc.get(&coord, M));
  EAR_TRY(sc.get(&roots, 1));
  EAR_CUDA_TRY(dev_memset(intree, 0, sizeof(int32_t) * (size_t)std::max<int64_t>(M, 1), st));
  EAR_CUDA_TRY(dev_memset(roots, 0, sizeof(int32_t), st));
  EAR_LAUNCH(k_mark_tree, grid_for(N), NT, 0, st)(N, lab, m->PE, intree, roots);
  int32_t f = 0;
  if (M > 0) {
    EAR_LAUNCH(k_not, grid_for(M), NT, 0, st)(M, intree, nflag);
    EAR_TRY(exclusive_sum(nflag, npos, M, sc));
    EAR_LAUNCH(k_coord, grid_for(M), NT, 0, st)(M, intree, npos, coord);
    int32_t lp = 0, lf = 0;
    EAR_TRY(read1(&lp, npos + M - 1, st));
    EAR_TRY(read1(&lf, nflag + M - 1, st));
    f = lp + lf;
  }
  int4 *ord4 = nullptr;
  EAR_TRY(sc.get(&ord4, NN));
  EAR_LAUNCH(k_order4, grid_for(NN), NT, 0, st)(N, L, order, lstart, m->PE, m->eu, m->ev, coord, ord4);
  EAR_TRY(read1(&m->k, roots, st));
  m->f = f;
  if ((int64_t)f != M - N + m->k) {
    set_error("ear_mcb: %d witness coordinates for M - N + k = %lld", f, (long long)(M - N + m->k));
    return EAR_ECUDA;
  }
  EAR_TRY(alloc_keep(&m->cyc_z, f, st));
  EAR_TRY(alloc_keep(&m->cyc_e, f, st));
  EAR_TRY(alloc_keep(&m->cyc_w, f, st));
  if (f == 0) return EAR_OK;
  // ---- candidates, sorted by (weight, perturbation)
  unsigned long long *cnt = nullptr;
  EAR_TRY(sc.get(&cnt, 1));
  EAR_CUDA_TRY(dev_memset(cnt, 0, sizeof(unsigned long long), st));
  const int64_t NM = (int64_t)N * M;
  EAR_LAUNCH(k_candidates, grid_for(NM), NT, 0, st)(N, M, Np, D, m->eu, m->ev, m->ew, m->PE, BR, H, cnt, nullptr,
                                                    nullptr);
  unsigned long long nc = 0;
  EAR_TRY(read1(&nc, cnt, st));
  m->ncand = (int64_t)nc;
  uint64_t *k0 = nullptr, *k1 = nullptr;
  int64_t *v0 = nullptr, *v1 = nullptr;
  EAR_TRY(sc.get(&k0, m->ncand));
  EAR_TRY(sc.get(&k1, m->ncand));
  EAR_TRY(sc.get(&v0, m->ncand));
  EAR_TRY(sc.get(&v1, m->ncand));
  EAR_CUDA_TRY(dev_memset(cnt, 0, sizeof(unsigned long long), st));
  EAR_LAUNCH(k_candidates, grid_for(NM), NT, 0, st)(N, M, Np, D, m->eu, m->ev, m->ew, m->PE, BR, H, cnt, k0, v0);
  // k_candidates emits in atomic order and equal keys (one cycle found from several roots) are common:
  // order by (z, e) first, then the stable sort by key leaves every tie in that order -- the same basis,
  // with the same root per cycle, on every run
  cub::DoubleBuffer<uint64_t> dk(k0, k1);
  cub::DoubleBuffer<int64_t> dv(v0, v1);
  {
    uint64_t *u0 = reinterpret_cast<uint64_t *>(v0), *u1 = reinterpret_cast<uint64_t *>(v1);
    int64_t *s0 = reinterpret_cast<int64_t *>(k0), *s1 = reinterpret_cast<int64_t *>(k1);
    cub::DoubleBuffer<uint64_t> dz(u0, u1);   // (z, e) as the key, the candidate key as the value
    cub::DoubleBuffer<int64_t> dy(s0, s1);
    size_t tb = 0, tb2 = 0;
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, m->ncand, 0, 64, st));
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb2, dz, dy, m->ncand, 0, 64, st));
    char *tmp = nullptr;
    EAR_TRY(sc.get(&tmp, (int64_t)std::max(tb, tb2)));
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb2, dz, dy, m->ncand, 0, 64, st));
    dk = cub::DoubleBuffer<uint64_t>(reinterpret_cast<uint64_t *>(dy.Current()),
                                     reinterpret_cast<uint64_t *>(dy.Alternate()));
    dv = cub::DoubleBuffer<int64_t>(reinterpret_cast<int64_t *>(dz.Current()),
                                    reinterpret_cast<int64_t *>(dz.Alternate()));
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dv, m->ncand, 0, 64, st));
  }
  // ---- phases
  const int32_t Wd = (f + 31) / 32, Wn = (N + 31) / 32;
  uint32_t *S = nullptr, *C = nullptr, *Lbits = nullptr;
  PhaseState *ps = nullptr;
  EAR_TRY(sc.get(&S, (int64_t)f * Wd));
  EAR_TRY(sc.get(&C, Wd));
  EAR_TRY(sc.get(&Lbits, (int64_t)N * Wn));
  EAR_TRY(sc.get(&ps, 1));
  EAR_LAUNCH(k_witness_init, grid_for((int64_t)f * Wd), NT, 0, st)(f, Wd, S);
  EAR_LAUNCH(k_ps_init, 1, 1, 0, st)(ps);
  const int lsmem = LW * Wn * 4;
  EAR_CUDA_TRY(smem_attr((const void *)k_labels, lsmem));
  const int scan_grid = num_sms() * 4;
  const int upd_grid = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div((int64_t)f * 32, NT), 148 * 8));
  for (int32_t i = 0; i < f; ++i) {
    const uint32_t *Si = S + (int64_t)i * Wd;
    EAR_LAUNCH(k_labels, (int)ceil_div(N, LW), LW * 32, lsmem, st)(N, L, ord4, lstart, Si, Lbits, Wn);
    EAR_LAUNCH(k_scan, scan_grid, NT, 0, st)(m->ncand, dv.Current(), m->eu, m->ev, coord, Si, Lbits, Wn, ps);
    EAR_LAUNCH(k_cycle, 1, 128, 0, st)(i, dk.Current(), dv.Current(), m->eu, m->ev, m->PE, coord, N, C, Wd, ps,
                                       m->cyc_z, m->cyc_e, m->cyc_w);
    EAR_LAUNCH(k_update, upd_grid, NT, 0, st)(i, f, Wd, S, C, ps);
  }
  PhaseState h{};
  EAR_TRY(read1(&h, ps, st));
  if (h.missing) {
    set_error("ear_mcb: a phase found no candidate non-orthogonal to its witness");
    return EAR_ECUDA;
  }
  m->weight = h.weight;
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

}  // namespace
}  // namespace ear

using namespace ear;

extern "C" {

ear_status_t ear_mcb(int32_t n, int64_t m, const int32_t *d_src, const int32_t *d_dst, const int32_t *d_w, void *stream,
                     ear_mcb_t *out) {
  NvtxRange nvtx_("ear: minimum cycle basis");
  if (!out) { set_error("ear_mcb: out is NULL"); return EAR_EINVAL; }
  *out = nullptr;
  if (n < 1 || m < 0 || (m > 0 && (!d_src || !d_dst || !d_w))) {
    set_error("ear_mcb: bad sizes n=%d m=%lld", n, (long long)m);
    return EAR_EINVAL;
  }
  ear_mcb_s *mc = new ear_mcb_s;
  ear_status_t s = mcb_build(mc, n, m, d_src, d_dst, d_w, (cudaStream_t)stream);
  if (s != EAR_OK) {
    cudaStreamSynchronize((cudaStream_t)stream);
    mcb_free(mc);
    delete mc;
    return s;
  }
  *out = mc;
  return EAR_OK;
}

ear_status_t ear_mcb_info(ear_mcb_t mc, ear_mcb_info_t *info) {
  if (!mc || !info) { set_error("ear_mcb_info: NULL argument"); return EAR_EINVAL; }
  info->dim = mc->f;
  info->weight = mc->weight;
  info->n_reduced = mc->N;
  info->m_reduced = mc->M;
  info->components = mc->k;
  info->n_candidates = mc->ncand;
  info->tree_depth = mc->dmax;
  return EAR_OK;
}

ear_status_t ear_mcb_cycle_weights(ear_mcb_t mc, int64_t *d_weights, void *stream) {
  if (!mc || (!d_weights && mc->f > 0)) { set_error("ear_mcb_cycle_weights: NULL argument"); return EAR_EINVAL; }
  if (mc->f > 0)
    EAR_CUDA_TRY(dev_copy(d_weights, mc->cyc_w, sizeof(int64_t) * (size_t)mc->f, (cudaStream_t)stream));
  return EAR_OK;
}

ear_status_t ear_mcb_cycle(ear_mcb_t mc, int32_t i, int32_t *d_verts, int32_t cap, int32_t *len, void *stream) {
  if (!mc || !len || i < 0 || i >= mc->f || cap < 0 || (cap > 0 && !d_verts)) {
    set_error("ear_mcb_cycle: bad argument (i=%d of %d)", i, mc ? mc->f : 0);
    return EAR_EINVAL;
  }
  cudaStream_t st = (cudaStream_t)stream;
  Scratch sc{st, {}};
  int32_t *dlen = nullptr, *scr = nullptr;
  EAR_TRY(sc.get(&dlen, 1));
  EAR_TRY(sc.get(&scr, mc->N + 1));
  EAR_LAUNCH(k_expand_cycle, 1, 32, 0, st)(i, mc->N, mc->cyc_z, mc->cyc_e, mc->eu, mc->ev, mc->ech, mc->PE,
                                           mc->plan->seg_start, mc->plan->seg_vert, mc->tid2v, d_verts, cap, dlen,
                                           scr);
  EAR_TRY(read1(len, dlen, st));
  return EAR_OK;
}

void ear_mcb_destroy(ear_mcb_t mc) {
  if (!mc) return;
  mcb_free(mc);
  delete mc;
}

}  // extern "C"
