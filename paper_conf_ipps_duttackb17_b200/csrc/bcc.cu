// Phase II over the biconnected components of G^r (paper sec. 2.2 "Extension to General Graphs",
// P:119-131).  Large sparse graphs are rarely 2-connected; the paper
// partitions G into its blocks G_1, G_2, ..., solves each block separately and joins the results
// through the articulation points with the block-cut tree:
//   d(n1, n2) = d(n1, a1) + d(a1, a2) + d(a2, n2)
// for n1, n2 in different blocks, a1 / a2 the articulation points on the way.
//
// B200 form (readings C21-C23 in DESIGN.md).  The chains are already contracted (Phase I), so the
// blocks are those of the simple reduced graph G^r (parallel G^r edges merged, P:90 -- distances are
// those of the multigraph).  Per connected component the LARGEST block is the root piece R; every
// other vertex v hangs off R through one vertex att(v) of R (the articulation point where its branch of
// the block-cut tree meets R), and the vertices hanging at a, with a, form the hanging piece H_a.  Then
//   same piece H_a   : S^r[u,v] = S_{H_a}[u,v]                  (a shortest path never leaves H_a:
//                                                                 it would re-enter through a)
//   otherwise        : S^r[u,v] = h(u) + S_R[att(u), att(v)] + h(v),   h(x) = S_{H_att(x)}[x, att(x)]
//   other component  : EAR_INF
// which is P:131 with the block-cut path collapsed onto the root block.  The FW work drops from N_r^3
// to n_R^3 + sum |H_a|^3; every piece is solved by a min-plus Floyd-Warshall of its own (one CTA per
// piece of <= 128 vertices in shared memory; the blocked TMA kernel for larger ones), and one compose
// kernel writes S^r into the caller's D, so Phase III is unchanged.
//
// The blocks themselves are found on the device with the Tarjan-Vishkin construction: a BFS spanning
// forest, preorder numbers / subtree sizes and low/high values by level sweeps (one CTA: the sweeps
// are latency bound and short), the auxiliary graph on tree edges, and its connected components by
// min-label hooking + pointer jumping.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "common.cuh"

struct ear_bcc_s {
  int32_t P = 0;                    // number of ranks the piece layout was padded for
  int32_t n_components = 0, n_blocks = 0, n_articulation = 0, n_pieces = 0, largest = 0, levels = 0;
  double sum_cubes = 0;
  int32_t *att = nullptr;           // [nr] attachment vertex in the root piece
  int32_t *ridx = nullptr;          // [nr] local index in the component's root piece, -1 if not in it
  int32_t *hp = nullptr;            // [nr] hanging piece at att(v), -1 if none
  int4 *cinfo = nullptr;            // [nr] {root piece, local index of att(v) in it, local index in hp, h(v)}
  int4 *arcs = nullptr;             // [A] {piece, local u, local x, w} for every arc of G^r
  int32_t n_arcs = 0;
  int32_t *psize = nullptr, *pld = nullptr;   // [np]
  int64_t *pbase = nullptr;                   // [np] offset of the piece matrix in the pool (ints)
  int64_t pool_ints = 0;
  std::vector<int32_t> h_psize, h_pld;
  std::vector<int64_t> h_pbase;
  std::vector<int32_t> big;                   // pieces with more than 128 vertices (blocked FW)
  int32_t rereduced = 0, largest_reduced = 0;  // last solve: big pieces reduced again, largest's size
  int32_t rereduce_levels = 0;                 // most nested reductions applied to one piece
};

namespace ear {

void bcc_free(ear_bcc_s *b, cudaStream_t st) {
  if (!b) return;
  void *arrs[] = {b->att, b->ridx, b->hp, b->cinfo, b->arcs, b->psize, b->pld, b->pbase};
  for (void *q : arrs)
    if (q) cudaFreeAsync(q, st);
  delete b;
}

namespace {

constexpr int NT = 256;
constexpr int TB = 1024;   // the single-CTA tree kernel
constexpr int SMALL = 128; // pieces up to this size: one CTA, shared-memory FW

#define GS(i, n) for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (n); i += (int64_t)gridDim.x * blockDim.x)

int grid_for(int64_t n) { return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, NT), 148 * 16)); }

// ------------------------------------------------------------------ connected components
// min-label hooking of roots + full pointer jumping; par[v] <= v always, so no cycles; at the fixed
// point par[v] = minimum vertex id of v's component.
__global__ void k_iota(int32_t *p, int32_t n) { GS(v, n) p[v] = (int32_t)v; }

__global__ void k_cc_hook(const int2 *e, const int32_t *ne, int32_t *par, int32_t *changed) {
  const int64_t m = *ne;
  GS(i, m) {
    const int2 x = e[i];
    const int32_t a = par[x.x], b = par[x.y];
    if (a != b) {
      atomicMin(&par[max(a, b)], min(a, b));
      *changed = 1;
    }
  }
}

__global__ void k_cc_jump(int32_t *par, int32_t n) {
  GS(v, n) {
    int32_t p = par[v];
    while (p != par[p]) p = par[p];
    par[v] = p;
  }
}

// ------------------------------------------------------------------ edge lists
__global__ void k_edges_all(const int32_t *rp, const int32_t *col, int32_t nr, int2 *e, int32_t *ne) {
  GS(u, nr) {
    for (int32_t a = rp[u]; a < rp[u + 1]; ++a) {
      const int32_t x = col[a];
      if ((int32_t)u < x) e[atomicAdd(ne, 1)] = make_int2((int32_t)u, x);
    }
  }
}

// Tarjan-Vishkin auxiliary graph on tree edges (identified by their child vertex):
//   (p(v), v) ~ (p(p), p)   if low(v) < pre(p) or high(v) >= pre(p) + size(p)   (p not a root)
//   (p(u), u) ~ (p(x), x)   for every non-tree edge (u, x) with u, x unrelated in the tree
__global__ void k_edges_aux(const int32_t *rp, const int32_t *col, int32_t nr, const int32_t *parent,
                            const int32_t *pre, const int32_t *size, const int32_t *low, const int32_t *high, int2 *e,
                            int32_t *ne) {
  GS(u, nr) {
    const int32_t p = parent[u];
    if (p >= 0 && parent[p] >= 0 && (low[u] < pre[p] || high[u] >= pre[p] + size[p]))
      e[atomicAdd(ne, 1)] = make_int2((int32_t)u, p);
    const int32_t pu = pre[u], su = size[u];
    for (int32_t a = rp[u]; a < rp[u + 1]; ++a) {
      const int32_t x = col[a];
      if ((int32_t)u >= x || parent[x] == (int32_t)u || p == x) continue;
      const int32_t px = pre[x], sx = size[x];
      const bool related = (pu <= px && px < pu + su) || (px <= pu && pu < px + sx);
      if (!related) e[atomicAdd(ne, 1)] = make_int2((int32_t)u, x);
    }
  }
}

// block label of the G^r edge (u, x)
__device__ __forceinline__ int32_t edge_block(int32_t u, int32_t x, const int32_t *parent, const int32_t *pre,
                                              const int32_t *blk) {
  if (parent[x] == u) return blk[x];
  if (parent[u] == x) return blk[u];
  return blk[pre[u] > pre[x] ? u : x];
}

// edges outside the root block of their component
__global__ void k_edges_rest(const int32_t *rp, const int32_t *col, int32_t nr, const int32_t *parent,
                             const int32_t *pre, const int32_t *blk, const int32_t *cc, const int32_t *rblock, int2 *e,
                             int32_t *ne) {
  GS(u, nr) {
    const int32_t R = rblock[cc[u]];
    for (int32_t a = rp[u]; a < rp[u + 1]; ++a) {
      const int32_t x = col[a];
      if ((int32_t)u < x && edge_block((int32_t)u, x, parent, pre, blk) != R) e[atomicAdd(ne, 1)] = make_int2((int32_t)u, x);
    }
  }
}

// ------------------------------------------------------------------ BFS root per component
// The level sweeps of k_tree cost one barrier-separated step per BFS level, so the root should be central:
// with spatially coherent labels the min-id vertex (the component label) sits at a corner and the BFS
// depth is the hop diameter.  Heuristic (any root gives the same blocks): the vertex whose id is closest
// to the middle of the component's id range [cc, max id].
__global__ void k_comp_maxid(int32_t nr, const int32_t *cc, int32_t *cmax) { GS(v, nr) atomicMax(&cmax[cc[v]], (int32_t)v); }
__global__ void k_comp_root(int32_t nr, const int32_t *cc, const int32_t *cmax, unsigned long long *rootkey) {
  GS(v, nr) {
    const int32_t c = cc[v];
    const int64_t mid = ((int64_t)c + cmax[c]) / 2, d = (int64_t)v >= mid ? (int64_t)v - mid : mid - (int64_t)v;
    atomicMin(&rootkey[c], ((unsigned long long)d << 32) | (uint32_t)v);
  }
}

// ------------------------------------------------------------------ spanning forest (one CTA)
// BFS from every component's root (k_comp_root), then subtree sizes (bottom-up), preorder numbers
// (top-down: children of u get consecutive ranges after pre(u)), and low/high = min/max preorder
// number reachable from the subtree through one non-tree edge (bottom-up).  Levels are separated by
// __syncthreads(), which also orders the global-memory atomics of the single block.
__global__ void __launch_bounds__(TB, 1)
    k_tree(int32_t nr, const int32_t *rp, const int32_t *col, const int32_t *cc, const unsigned long long *rootkey,
           int32_t *parent, int32_t *order, int32_t *lvl, int32_t *size, int32_t *pre, int32_t *low, int32_t *high,
           int32_t *out_levels) {
  using BS = cub::BlockScan<int32_t, TB>;
  __shared__ typename BS::TempStorage ts;
  __shared__ int32_t s_tail, s_carry;
  const int t = threadIdx.x;
  for (int32_t v = t; v < nr; v += TB) {
    parent[v] = (int32_t)(uint32_t)rootkey[cc[v]] == v ? -1 : -2;
    size[v] = 1;
  }
  if (t == 0) s_carry = 0;
  __syncthreads();
  for (int32_t b0 = 0; b0 < nr; b0 += TB) {   // roots, ascending
    const int32_t v = b0 + t;
    const int32_t f = (v < nr && (int32_t)(uint32_t)rootkey[cc[v]] == v) ? 1 : 0;
    int32_t off, tot;
    BS(ts).ExclusiveSum(f, off, tot);
    if (f) order[s_carry + off] = v;
    __syncthreads();
    if (t == 0) s_carry += tot;
    __syncthreads();
  }
  const int32_t R = s_carry;
  if (t == 0) {
    s_tail = R;
    lvl[0] = 0;
    lvl[1] = R;
  }
  __syncthreads();
  // BFS: level l = order[lvl[l] .. lvl[l+1])
  int32_t nl = 1, b = 0, e = R;
  while (true) {
    for (int32_t i = b + t; i < e; i += TB) {
      const int32_t u = order[i];
      for (int32_t a = rp[u]; a < rp[u + 1]; ++a) {
        const int32_t x = col[a];
        if (atomicCAS(&parent[x], -2, u) == -2) order[atomicAdd(&s_tail, 1)] = x;
      }
    }
    __syncthreads();
    const int32_t ne = s_tail;
    __syncthreads();
    if (ne == e) break;
    if (t == 0) lvl[nl + 1] = ne;
    ++nl;
    b = e;
    e = ne;
  }
  __syncthreads();
  // subtree sizes
  for (int32_t l = nl - 1; l >= 1; --l) {
    for (int32_t i = lvl[l] + t; i < lvl[l + 1]; i += TB) {
      const int32_t v = order[i];
      atomicAdd(&size[parent[v]], size[v]);
    }
    __syncthreads();
  }
  // preorder numbers: roots by an exclusive scan of their sizes, then top-down
  if (t == 0) s_carry = 0;
  __syncthreads();
  for (int32_t b0 = 0; b0 < R; b0 += TB) {
    const int32_t i = b0 + t;
    const int32_t s = i < R ? size[order[i]] : 0;
    int32_t off, tot;
    BS(ts).ExclusiveSum(s, off, tot);
    if (i < R) pre[order[i]] = s_carry + off;
    __syncthreads();
    if (t == 0) s_carry += tot;
    __syncthreads();
  }
  for (int32_t l = 0; l + 1 < nl; ++l) {
    for (int32_t i = lvl[l] + t; i < lvl[l + 1]; i += TB) {
      const int32_t u = order[i];
      int32_t run = pre[u] + 1;
      for (int32_t a = rp[u]; a < rp[u + 1]; ++a) {
        const int32_t x = col[a];
        if (parent[x] == u) {
          pre[x] = run;
          run += size[x];
        }
      }
    }
    __syncthreads();
  }
  // low / high
  for (int32_t v = t; v < nr; v += TB) {
    int32_t lo = pre[v], hi = pre[v];
    const int32_t p = parent[v];
    for (int32_t a = rp[v]; a < rp[v + 1]; ++a) {
      const int32_t x = col[a];
      if (x == p || parent[x] == v) continue;
      lo = min(lo, pre[x]);
      hi = max(hi, pre[x]);
    }
    low[v] = lo;
    high[v] = hi;
  }
  __syncthreads();
  for (int32_t l = nl - 1; l >= 1; --l) {
    for (int32_t i = lvl[l] + t; i < lvl[l + 1]; i += TB) {
      const int32_t v = order[i];
      atomicMin(&low[parent[v]], low[v]);
      atomicMax(&high[parent[v]], high[v]);
    }
    __syncthreads();
  }
  if (t == 0) *out_levels = nl;
}

// ------------------------------------------------------------------ blocks, root blocks, pieces
// aux component root -> block id of every tree edge; roots of the spanning forest get -1
__global__ void k_block_stats(int32_t nr, const int32_t *parent, int32_t *blk, int32_t *bcnt, int32_t *top) {
  GS(v, nr) {
    const int32_t p = parent[v];
    if (p < 0) continue;
    const int32_t b = blk[v];
    atomicAdd(&bcnt[b], 1);
    if (parent[p] < 0 || blk[p] != b) top[b] = p;
  }
}

__global__ void k_root_blocks(int32_t nr, const int32_t *parent, const int32_t *blk, const int32_t *bcnt,
                              const int32_t *top, const int32_t *cc, unsigned long long *rkey, int32_t *ntop,
                              int32_t *counts /* [0] blocks */) {
  GS(v, nr) {
    if (parent[v] < 0 || blk[v] != (int32_t)v) continue;   // v names its block
    atomicAdd(&counts[0], 1);
    atomicAdd(&ntop[top[v]], 1);
    const unsigned long long key = ((unsigned long long)(bcnt[v] + 1) << 32) | (uint32_t)(0x7FFFFFFF - (int32_t)v);
    atomicMax(&rkey[cc[v]], key);
  }
}

__global__ void k_root_of_comp(int32_t nr, const int32_t *cc, const int32_t *parent, const int32_t *ntop,
                               const unsigned long long *rkey, int32_t *rblock, int32_t *counts /* [1] comps, [2] APs */) {
  GS(v, nr) {
    if (cc[v] == (int32_t)v) {
      atomicAdd(&counts[1], 1);
      rblock[v] = rkey[v] ? (int32_t)(0x7FFFFFFF - (uint32_t)(rkey[v] & 0xFFFFFFFFu)) : -1;
    }
    if ((parent[v] >= 0 && ntop[v] >= 1) || (parent[v] < 0 && ntop[v] >= 2)) atomicAdd(&counts[2], 1);
  }
}

__device__ __forceinline__ bool in_root(int32_t v, const int32_t *cc, const int32_t *rblock, const int32_t *blk,
                                        const int32_t *top) {
  const int32_t R = rblock[cc[v]];
  return R < 0 || blk[v] == R || top[R] == v;
}

__global__ void k_attach(int32_t nr, const int32_t *cc, const int32_t *rblock, const int32_t *blk, const int32_t *top,
                         const int32_t *rc, int32_t *att_of, int32_t *hsz) {
  GS(v, nr) {
    if (in_root((int32_t)v, cc, rblock, blk, top)) att_of[rc[v]] = (int32_t)v;
    atomicAdd(&hsz[rc[v]], 1);
  }
}

__device__ __forceinline__ int64_t round_up_d(int64_t a, int64_t b) { return (a + b - 1) / b * b; }

// pieces owned by vertex v: the root piece of its component (v == cc[v]) and the hanging piece of its
// remainder component (v == rc[v], >= 2 vertices)
__global__ void k_piece_count(int32_t nr, const int32_t *cc, const int32_t *rc, const int32_t *hsz, int32_t *cnt) {
  GS(v, nr) cnt[v] = (cc[v] == (int32_t)v) + (rc[v] == (int32_t)v && hsz[v] >= 2);
}

__global__ void k_piece_sizes(int32_t nr, const int32_t *cc, const int32_t *rc, const int32_t *hsz,
                              const int32_t *rblock, const int32_t *bcnt, const int32_t *pid0, int32_t P,
                              int32_t *psize, int32_t *pld, int64_t *palloc) {
  GS(v, nr) {
    int32_t id = pid0[v];
    auto put = [&](int32_t s) {
      const int32_t ld = s <= SMALL ? s : (int32_t)round_up_d(s, (int64_t)TILE * P);
      psize[id] = s;
      pld[id] = ld;
      palloc[id] = ((int64_t)ld * ld + 31) / 32 * 32;   // 128-byte aligned piece matrices
      ++id;
    };
    if (cc[v] == (int32_t)v) put(rblock[v] < 0 ? 1 : bcnt[rblock[v]] + 1);
    if (rc[v] == (int32_t)v && hsz[v] >= 2) put(hsz[v]);
  }
}

__global__ void k_member_keys(int32_t nr, const int32_t *cc, const int32_t *rblock, const int32_t *blk,
                              const int32_t *top, const int32_t *rc, const int32_t *hsz, const int32_t *pid0,
                              int32_t np, int32_t *keys, int32_t *vals) {
  GS(v, nr) {
    const int32_t c = cc[v], r = rc[v];
    keys[2 * v] = in_root((int32_t)v, cc, rblock, blk, top) ? pid0[c] : np;
    keys[2 * v + 1] = hsz[r] >= 2 ? pid0[r] + (cc[r] == r) : np;
    vals[2 * v] = vals[2 * v + 1] = (int32_t)v;
  }
}

__global__ void k_member_local(int64_t nm, const int32_t *keys, const int32_t *vals, const int32_t *pstart,
                               int32_t np, const int32_t *cc, const int32_t *pid0, int32_t *ridx, int32_t *hloc) {
  GS(i, nm) {
    const int32_t k = keys[i];
    if (k >= np) continue;
    const int32_t v = vals[i];
    const int32_t loc = (int32_t)i - pstart[k];
    if (k == pid0[cc[v]]) ridx[v] = loc;
    else hloc[v] = loc;
  }
}

__global__ void k_vertex_info(int32_t nr, const int32_t *cc, const int32_t *rc, const int32_t *hsz,
                              const int32_t *att_of, const int32_t *pid0, const int32_t *ridx, const int32_t *hloc,
                              int32_t *att, int32_t *hp, int4 *cinfo) {
  GS(v, nr) {
    const int32_t r = rc[v], a = att_of[r];
    att[v] = a;
    hp[v] = hsz[r] >= 2 ? pid0[r] + (cc[r] == r) : -1;
    cinfo[v] = make_int4(pid0[cc[v]], ridx[a], hloc[v], 0);
  }
}

__global__ void k_piece_arcs(const int32_t *rp, const int32_t *col, const int32_t *wt, int32_t nr,
                             const int32_t *parent, const int32_t *pre, const int32_t *blk, const int32_t *cc,
                             const int32_t *rblock, const int32_t *pid0, const int32_t *hp, const int32_t *ridx,
                             const int32_t *hloc, int4 *arcs) {
  GS(u, nr) {
    const int32_t R = rblock[cc[u]];
    for (int32_t a = rp[u]; a < rp[u + 1]; ++a) {
      const int32_t x = col[a];
      if (edge_block((int32_t)u, x, parent, pre, blk) == R) arcs[a] = make_int4(pid0[cc[u]], ridx[u], ridx[x], wt[a]);
      else arcs[a] = make_int4(hp[u], hloc[u], hloc[x], wt[a]);
    }
  }
}

// ------------------------------------------------------------------ per-solve kernels
__global__ void k_fill_pool(int32_t *p, int64_t n) {
  GS(i, n / 4) reinterpret_cast<int4 *>(p)[i] = make_int4(INF, INF, INF, INF);
  GS(i, n % 4) p[n / 4 * 4 + i] = INF;
}

__global__ void k_pool_init(int32_t nr, const int4 *cinfo, const int32_t *ridx, const int32_t *hp, const int32_t *pld,
                            const int64_t *pbase, const int4 *arcs, int32_t A, int32_t *pool) {
  GS(v, nr) {
    const int4 ci = cinfo[v];
    if (ridx[v] >= 0) pool[pbase[ci.x] + (int64_t)ridx[v] * (pld[ci.x] + 1)] = 0;
    if (ci.z >= 0) pool[pbase[hp[v]] + (int64_t)ci.z * (pld[hp[v]] + 1)] = 0;
  }
  GS(a, A) {
    const int4 e = arcs[a];
    pool[pbase[e.x] + (int64_t)e.y * pld[e.x] + e.z] = e.w;
  }
}

// the arcs of piece `pc` as a piece-local edge list (both directions; decompose() merges them)
__global__ void k_piece_edges(const int4 *arcs, int32_t A, int32_t pc, int32_t *u, int32_t *v, int32_t *w,
                              int32_t *cnt) {
  GS(a, A) {
    const int4 e = arcs[a];
    if (e.x == pc && e.y < e.z) {
      const int32_t i = atomicAdd(cnt, 1);
      u[i] = e.y; v[i] = e.z; w[i] = e.w;
    }
  }
}

// one CTA per piece of 3..128 vertices: plain Floyd-Warshall in shared memory (P:101 per block)
__global__ void __launch_bounds__(NT) k_piece_fw(int32_t np, const int32_t *psize, const int32_t *pld,
                                                 const int64_t *pbase, int32_t *pool) {
  extern __shared__ int32_t sd[];
  const int32_t p = blockIdx.x;
  const int32_t s = psize[p];
  if (s <= 2 || s > SMALL) return;
  int32_t *g = pool + pbase[p];   // ld == s for small pieces
  const int32_t ss = s * s;
  for (int32_t i = threadIdx.x; i < ss; i += NT) sd[i] = g[i];
  __syncthreads();
  for (int32_t k = 0; k < s; ++k) {
    for (int32_t i = threadIdx.x; i < ss; i += NT) {
      const int32_t r = i / s, c = i - r * s;
      const int32_t via = sd[r * s + k] + sd[k * s + c];
      if (via < sd[i]) sd[i] = via;
    }
    __syncthreads();
  }
  for (int32_t i = threadIdx.x; i < ss; i += NT) g[i] = sd[i];
}

// h(v) = S_{H_att(v)}[v, att(v)] into cinfo[v].w
__global__ void k_hang_dist(int32_t nr, const int32_t *att, const int32_t *hp, const int32_t *pld,
                            const int64_t *pbase, const int32_t *pool, int4 *cinfo) {
  GS(v, nr) {
    const int32_t a = att[v], h = hp[v];
    int32_t d = 0;
    if (a != (int32_t)v) d = pool[pbase[h] + (int64_t)cinfo[v].z * pld[h] + cinfo[a].z];
    cinfo[v].w = d;
  }
}

// S^r rows from the pieces: RB rows per CTA, 4 columns per thread (int4 stores)
constexpr int RB = 8;
// D16 (optional, rows of stride ld16, columns [0, ld16)): the same rows as u16 for the pair-major
// expansion, 0xFFFF = INF; a finite entry >= 0xFFFF sets *flag16.  D may be NULL when only D16 is wanted.
__global__ void __launch_bounds__(NT) k_compose(int32_t nr, int32_t Np, const int4 *__restrict__ cinfo,
                                                const int32_t *__restrict__ hp, const int32_t *__restrict__ pld,
                                                const int64_t *__restrict__ pbase, const int32_t *__restrict__ pool,
                                                int32_t *D, int64_t ldd, int32_t row0, int32_t rows,
                                                const int32_t *trows, uint16_t *D16, int64_t ld16, int32_t *flag16) {
  int over = 0;
  __shared__ int4 s_row[RB];                 // {root piece, ratt, hloc, h}
  __shared__ const int32_t *s_R[RB], *s_H[RB];
  __shared__ int32_t s_u[RB];
  for (int32_t g0 = blockIdx.x * RB; g0 < rows; g0 += gridDim.x * RB) {
    if (threadIdx.x < RB) {
      const int32_t lr = g0 + threadIdx.x;
      int32_t u = -1;
      if (lr < rows) u = trows ? trows[lr / TILE] * TILE + lr % TILE : row0 + lr;
      s_u[threadIdx.x] = u;
      if (u >= 0 && u < nr) {
        const int4 ci = cinfo[u];
        s_row[threadIdx.x] = ci;
        s_R[threadIdx.x] = pool + pbase[ci.x] + (int64_t)ci.y * pld[ci.x];
        const int32_t h = hp[u];
        s_H[threadIdx.x] = h >= 0 ? pool + pbase[h] + (int64_t)ci.z * pld[h] : nullptr;
      }
    }
    __syncthreads();
    for (int32_t c4 = threadIdx.x; c4 < Np / 4; c4 += NT) {
      int4 cv[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int32_t v = c4 * 4 + j;
        cv[j] = v < nr ? cinfo[v] : make_int4(-1, -1, -1, 0);
      }
#pragma unroll
      for (int r = 0; r < RB; ++r) {
        const int32_t u = s_u[r];
        if (g0 + r >= rows) break;
        int32_t o[4];
        if (u >= nr) {
#pragma unroll
          for (int j = 0; j < 4; ++j) o[j] = (c4 * 4 + j == u) ? 0 : INF;
        } else {
          const int4 ru = s_row[r];
          const int32_t *Rrow = s_R[r], *Hrow = s_H[r];
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const int32_t v = c4 * 4 + j;
            const int4 c = cv[j];
            int32_t d;
            if (c.x != ru.x) d = INF;                         // other component (or padding)
            else if (c.y == ru.y) d = v == u ? 0 : Hrow[c.z]; // same attachment: inside H_att
            else d = min(INF, ru.w + Rrow[c.y] + c.w);        // P:131 through the root piece
            o[j] = d;
          }
        }
        if (D) *reinterpret_cast<int4 *>(D + (int64_t)(g0 + r) * ldd + c4 * 4) = make_int4(o[0], o[1], o[2], o[3]);
        if (D16 && c4 * 4 < ld16) {
          uint32_t h[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            over |= o[j] >= 0xFFFF && o[j] < INF;
            h[j] = o[j] >= INF ? 0xFFFFu : (uint32_t)min(o[j], 0xFFFF);
          }
          *reinterpret_cast<uint2 *>(D16 + (int64_t)(g0 + r) * ld16 + c4 * 4) = make_uint2(h[0] | (h[1] << 16), h[2] | (h[3] << 16));
        }
      }
    }
    __syncthreads();
  }
  if (D16 && __syncthreads_or(over) && threadIdx.x == 0) atomicOr(flag16, 1);
}

struct Tmp {
  std::vector<void *> ptrs;
  cudaStream_t st;
  ~Tmp() {
    for (void *p : ptrs) cudaFreeAsync(p, st);
  }
  template <class T>
  T *get(int64_t count) {
    void *p = nullptr;
    if (cudaMallocAsync(&p, std::max<size_t>(16, sizeof(T) * (size_t)count), st) != cudaSuccess) return nullptr;
    ptrs.push_back(p);
    return (T *)p;
  }
};

ear_status_t cc_run(int32_t nv, const int2 *e, const int32_t *ne, int64_t ne_max, int32_t *par, int32_t *changed,
                    cudaStream_t st) {
  EAR_LAUNCH(k_iota, grid_for(nv), NT, 0, st)(par, nv);
  for (int it = 0; it < 4 * 32 + 8; ++it) {
    int32_t h = 0;
    EAR_CUDA_TRY(dev_memset(changed, 0, 4, st));
    EAR_LAUNCH(k_cc_hook, grid_for(ne_max), NT, 0, st)(e, ne, par, changed);
    EAR_LAUNCH(k_cc_jump, grid_for(nv), NT, 0, st)(par, nv);
    Readback rb(st);
    EAR_CUDA_TRY(rb.get(&h, changed, 4));
    EAR_CUDA_TRY(rb.sync());
    if (!h) return EAR_OK;
  }
  set_error("bcc: connected components did not converge");
  return EAR_ECUDA;
}

}  // namespace

ear_status_t sssp_prepare(ear_plan_s *p, cudaStream_t st);

// Block structure and piece layout of G^r (once per plan and rank count).  Synchronises `st`.
ear_status_t bcc_prepare(ear_plan_s *p, int32_t P, cudaStream_t st) {
  if (p->bcc && p->bcc->P == P) return EAR_OK;
  if (p->bcc) {
    bcc_free(p->bcc, st);
    p->bcc = nullptr;
  }
  EAR_TRY(sssp_prepare(p, st));
  const int32_t nr = p->n_reduced;
  const int32_t A = p->n_rarcs;
  const int32_t *rp = p->r_rowptr, *col = p->r_col, *wt = p->r_w;
  Tmp T{{}, st};
  int32_t *cc = T.get<int32_t>(nr), *rc = T.get<int32_t>(nr), *blk = T.get<int32_t>(nr);
  int32_t *parent = T.get<int32_t>(nr), *order = T.get<int32_t>(nr), *lvl = T.get<int32_t>(nr + 2);
  int32_t *size = T.get<int32_t>(nr), *pre = T.get<int32_t>(nr), *low = T.get<int32_t>(nr), *high = T.get<int32_t>(nr);
  int32_t *bcnt = T.get<int32_t>(nr), *top = T.get<int32_t>(nr), *ntop = T.get<int32_t>(nr);
  int32_t *rblock = T.get<int32_t>(nr), *att_of = T.get<int32_t>(nr), *hsz = T.get<int32_t>(nr);
  int32_t *cnt = T.get<int32_t>(nr + 1), *pid0 = T.get<int32_t>(nr + 1);
  int32_t *hloc = T.get<int32_t>(nr), *scal = T.get<int32_t>(8);
  unsigned long long *rkey = T.get<unsigned long long>(nr);
  int2 *e = T.get<int2>(std::max<int64_t>(A / 2, 1) + nr);
  int32_t *keys0 = T.get<int32_t>(2 * (int64_t)nr), *keys1 = T.get<int32_t>(2 * (int64_t)nr);
  int32_t *vals0 = T.get<int32_t>(2 * (int64_t)nr), *vals1 = T.get<int32_t>(2 * (int64_t)nr);
  if (!rkey || !e || !vals1 || !keys1 || !scal || !hloc) {
    set_error("bcc_prepare: out of device memory");
    return EAR_ENOMEM;
  }
  ear_bcc_s *b = new ear_bcc_s;
  b->P = P;
  p->bcc = b;
  auto dalloc = [&](void **q, size_t bytes) { return cudaMallocAsync(q, std::max<size_t>(bytes, 16), st); };
  if (dalloc((void **)&b->att, 4 * (size_t)nr) != cudaSuccess || dalloc((void **)&b->ridx, 4 * (size_t)nr) != cudaSuccess ||
      dalloc((void **)&b->hp, 4 * (size_t)nr) != cudaSuccess || dalloc((void **)&b->cinfo, 16 * (size_t)nr) != cudaSuccess ||
      dalloc((void **)&b->arcs, 16 * (size_t)A) != cudaSuccess) {
    set_error("bcc_prepare: out of device memory");
    return EAR_ENOMEM;
  }
  b->n_arcs = A;
  int32_t *ne = scal, *changed = scal + 1, *counts = scal + 2, *levels = scal + 6;
  EAR_CUDA_TRY(dev_memset(scal, 0, 32, st));
  const int64_t emax = std::max<int64_t>(A / 2, 1) + nr;
  // 1. connected components
  EAR_LAUNCH(k_edges_all, grid_for(nr), NT, 0, st)(rp, col, nr, e, ne);
  EAR_TRY(cc_run(nr, e, ne, emax, cc, changed, st));
  // 2. spanning forest, preorder, low/high
  // rkey and size are scratch here (both are initialised again below / inside k_tree)
  EAR_CUDA_TRY(dev_memset(size, 0, 4 * (size_t)nr, st));
  EAR_CUDA_TRY(dev_memset(rkey, 0xFF, 8 * (size_t)nr, st));
  EAR_LAUNCH(k_comp_maxid, grid_for(nr), NT, 0, st)(nr, cc, size);
  EAR_LAUNCH(k_comp_root, grid_for(nr), NT, 0, st)(nr, cc, size, rkey);
  EAR_LAUNCH(k_tree, 1, TB, 0, st)(nr, rp, col, cc, rkey, parent, order, lvl, size, pre, low, high, levels);
  // 3. auxiliary graph -> blocks
  EAR_CUDA_TRY(dev_memset(ne, 0, 4, st));
  EAR_LAUNCH(k_edges_aux, grid_for(nr), NT, 0, st)(rp, col, nr, parent, pre, size, low, high, e, ne);
  EAR_TRY(cc_run(nr, e, ne, emax, blk, changed, st));
  EAR_CUDA_TRY(dev_memset(bcnt, 0, 4 * (size_t)nr, st));
  EAR_CUDA_TRY(dev_memset(ntop, 0, 4 * (size_t)nr, st));
  EAR_CUDA_TRY(dev_memset(rkey, 0, 8 * (size_t)nr, st));
  EAR_LAUNCH(k_block_stats, grid_for(nr), NT, 0, st)(nr, parent, blk, bcnt, top);
  EAR_LAUNCH(k_root_blocks, grid_for(nr), NT, 0, st)(nr, parent, blk, bcnt, top, cc, rkey, ntop, counts);
  EAR_LAUNCH(k_root_of_comp, grid_for(nr), NT, 0, st)(nr, cc, parent, ntop, rkey, rblock, counts);
  // 4. the remainder graph (edges outside the root blocks) -> hanging pieces and attachments
  EAR_CUDA_TRY(dev_memset(ne, 0, 4, st));
  EAR_LAUNCH(k_edges_rest, grid_for(nr), NT, 0, st)(rp, col, nr, parent, pre, blk, cc, rblock, e, ne);
  EAR_TRY(cc_run(nr, e, ne, emax, rc, changed, st));
  EAR_CUDA_TRY(dev_memset(hsz, 0, 4 * (size_t)nr, st));
  EAR_LAUNCH(k_attach, grid_for(nr), NT, 0, st)(nr, cc, rblock, blk, top, rc, att_of, hsz);
  // 5. pieces: ids, sizes, layout
  EAR_LAUNCH(k_piece_count, grid_for(nr), NT, 0, st)(nr, cc, rc, hsz, cnt);
  size_t tb = 0, tb2 = 0, tb3 = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, pid0, nr + 1, st);
  void *tmp = T.get<char>((int64_t)tb);
  EAR_CUDA_TRY(dev_memset(cnt + nr, 0, 4, st));
  EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb, cnt, pid0, nr + 1, st));
  int32_t np = 0, hcounts[8] = {0};
  {
    Readback rb(st);
    EAR_CUDA_TRY(rb.get(&np, pid0 + nr, 4));
    EAR_CUDA_TRY(rb.get(hcounts, scal, 32));
    EAR_CUDA_TRY(rb.sync());
  }
  b->n_blocks = hcounts[2];
  b->n_components = hcounts[3];
  b->n_articulation = hcounts[4];
  b->levels = hcounts[6];
  b->n_pieces = np;
  int64_t *palloc = T.get<int64_t>(np + 1);
  int32_t *pstart = T.get<int32_t>(np + 1);
  if (dalloc((void **)&b->psize, 4 * (size_t)(np + 1)) != cudaSuccess ||
      dalloc((void **)&b->pld, 4 * (size_t)(np + 1)) != cudaSuccess ||
      dalloc((void **)&b->pbase, 8 * (size_t)(np + 1)) != cudaSuccess || !palloc || !pstart) {
    set_error("bcc_prepare: out of device memory");
    return EAR_ENOMEM;
  }
  EAR_CUDA_TRY(dev_memset(palloc + np, 0, 8, st));
  EAR_CUDA_TRY(dev_memset(b->psize + np, 0, 4, st));
  EAR_LAUNCH(k_piece_sizes, grid_for(nr), NT, 0, st)(nr, cc, rc, hsz, rblock, bcnt, pid0, P, b->psize, b->pld, palloc);
  cub::DeviceScan::ExclusiveSum(nullptr, tb2, palloc, b->pbase, np + 1, st);
  cub::DeviceScan::ExclusiveSum(nullptr, tb3, b->psize, pstart, np + 1, st);
  size_t tbs = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, tbs, keys0, keys1, vals0, vals1, (int)(2 * (int64_t)nr), 0, 32, st);
  void *tmp2 = T.get<char>((int64_t)std::max({tb2, tb3, tbs}));
  if (!tmp2) { set_error("bcc_prepare: out of device memory"); return EAR_ENOMEM; }
  EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp2, tb2, palloc, b->pbase, np + 1, st));
  EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp2, tb3, b->psize, pstart, np + 1, st));
  // local indices: memberships sorted by piece (stable: ascending vertex id inside a piece)
  EAR_LAUNCH(k_member_keys, grid_for(nr), NT, 0, st)(nr, cc, rblock, blk, top, rc, hsz, pid0, np, keys0, vals0);
  int bits = 1;
  while ((1ll << bits) <= np) ++bits;
  EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp2, tbs, keys0, keys1, vals0, vals1, (int)(2 * (int64_t)nr), 0, bits, st));
  EAR_CUDA_TRY(dev_memset(b->ridx, 0xFF, 4 * (size_t)nr, st));
  EAR_CUDA_TRY(dev_memset(hloc, 0xFF, 4 * (size_t)nr, st));
  EAR_LAUNCH(k_member_local, grid_for(2 * (int64_t)nr), NT, 0, st)(2 * (int64_t)nr, keys1, vals1, pstart, np, cc, pid0,
                                                                  b->ridx, hloc);
  EAR_LAUNCH(k_vertex_info, grid_for(nr), NT, 0, st)(nr, cc, rc, hsz, att_of, pid0, b->ridx, hloc, b->att, b->hp,
                                                     b->cinfo);
  if (A > 0)
    EAR_LAUNCH(k_piece_arcs, grid_for(nr), NT, 0, st)(rp, col, wt, nr, parent, pre, blk, cc, rblock, pid0, b->hp,
                                                      b->ridx, hloc, b->arcs);
  b->h_psize.resize(np);
  b->h_pld.resize(np);
  b->h_pbase.resize(np + 1);
  {
    Readback rb(st);
    EAR_CUDA_TRY(rb.get(b->h_psize.data(), b->psize, 4 * (size_t)np));
    EAR_CUDA_TRY(rb.get(b->h_pld.data(), b->pld, 4 * (size_t)np));
    EAR_CUDA_TRY(rb.get(b->h_pbase.data(), b->pbase, 8 * (size_t)(np + 1)));
    EAR_CUDA_TRY(rb.sync());
  }
  EAR_CUDA_TRY(cudaGetLastError());
  b->pool_ints = b->h_pbase[np];
  b->largest = 0;
  b->sum_cubes = 0;
  for (int32_t i = 0; i < np; ++i) {
    b->largest = std::max(b->largest, b->h_psize[i]);
    b->sum_cubes += (double)b->h_psize[i] * b->h_psize[i] * b->h_psize[i];
    if (b->h_psize[i] > SMALL) b->big.push_back(i);
  }
  std::sort(b->big.begin(), b->big.end(), [&](int32_t x, int32_t y) { return b->h_psize[x] > b->h_psize[y]; });
  return EAR_OK;
}


// The paper's order inside a big piece (G is split into its biconnected components and EACH is
// then reduced): a vertex of degree >= 3 in G^r can have degree 2 inside its block (an articulation
// point with one edge to a hanging piece), so the piece is reduced again -- Phase I on the piece's
// local edge list -- and the piece matrix M (ld, piece-local ids) is Phase III of that reduction over
// the FW of the smaller reduced piece.  Used when the reduced piece needs fewer 128-tiles; *done =
// false leaves M for the FW on the whole piece.  With a communicator the reduced
// piece is row-block sharded and gathered, and every rank expands M (all ranks need the whole piece).
constexpr int REREDUCE_DEPTH = 4;

// Distance matrix M (n x n, ld) of a connected graph given as an edge list, by the paper's method
// applied to it: Reduce (Phase I) -> distances of the reduced graph -> UPDATE_DISTANCE (Phase III).
// The reduced graph's distances come from the same recursion when its own Reduce still saves a tile
// (merging parallel edges can leave new degree-two vertices), else
// from the FW (sharded with a communicator).  *done = false (nothing written) when Reduce saves no
// tile at the top level.  *levels / *n_last: reductions applied and the size the FW ran on.
static ear_status_t reduce_solve(const ear_plan_s *p, int32_t n, int64_t m, const int32_t *u, const int32_t *v,
                                 const int32_t *w, int32_t *M, int64_t ld, ear_comm_s *comm, int depth,
                                 cudaStream_t st, bool *done, int32_t *levels, int32_t *n_last) {
  *done = false;
  ear_plan_s *q = new ear_plan_s;
  q->device = p->device;
  int sr = prof_begin(PK_REREDUCE, st);
  ear_status_t s = decompose(n, m, u, v, w, p->flags & EAR_FLAG_FW32, st, q);
  prof_end(sr, st, 0);
  // worth it when the FW runs on fewer 128-tiles (same tile count: same FW work, plus the expansion);
  // pieces solved by SSSP (EAR_FLAG_SSSP) always take the top level -- its plan is what the SSSP runs
  // on -- and a deeper one when it removes vertices
  const bool by_sssp = (p->flags & EAR_FLAG_SSSP) != 0;
  const int64_t unit = (int64_t)TILE * (comm ? comm->nranks : 1);
  const bool worth = s == EAR_OK && (by_sssp ? depth == 0 || q->n_reduced < n
                                             : round_up(std::max<int64_t>(q->n_reduced, 1), unit) < round_up(n, unit));
  if (s == EAR_OK && by_sssp && !comm && depth == 0 && (int64_t)q->n_reduced * 10 > (int64_t)n * 9) {
    // the contraction removes < 10 % of the piece: its Phase III pass (a gather per entry of the piece
    // matrix; cfg4's root piece: 4.2 ms for 405 vertices removed) costs more than the SSSP work it saves
    // (~n^2 scaling, 1.8 ms).  Run the SSSP on the piece itself instead -- every vertex a terminal, so
    // the plan's ids are the piece's own -- with the rows written straight into M.
    cudaStreamSynchronize(st);
    plan_free(q);
    delete q;
    q = new ear_plan_s;
    q->device = p->device;
    s = decompose(n, m, u, v, w, EAR_FLAG_NO_CONTRACT | (p->flags & EAR_FLAG_FW32), st, q);
    const int32_t Lp = (int32_t)round_up(std::max<int64_t>(n, 1), (int64_t)TILE);
    if (s == EAR_OK && ld >= Lp) s = sssp_rows(q, M, ld, Lp, 0, n, nullptr, st);
    else if (s == EAR_OK) s = EAR_EUNSUPPORTED;   // (pool matrices are padded to whole tiles)
    cudaStreamSynchronize(st);
    plan_free(q);
    delete q;
    if (s == EAR_OK) {
      *done = true;
      *levels = depth;
      *n_last = n;
    }
    return s;
  }
  if (!worth) {
    cudaStreamSynchronize(st);
    plan_free(q);
    delete q;
    return s;
  }
  *levels = depth + 1;
  *n_last = q->n_reduced;
  const int32_t P = comm ? comm->nranks : 1;
  const int32_t Np = (int32_t)round_up(std::max<int64_t>(q->n_reduced, 1), (int64_t)TILE * P);
  const bool allow16 = !(p->flags & EAR_FLAG_FW32);
  int32_t *D = nullptr;
  bool inner = false;
  if (cudaMallocAsync((void **)&D, sizeof(int32_t) * (size_t)Np * Np, st) != cudaSuccess) {
    set_error("bcc_solve: out of device memory (re-reduced piece)");
    s = EAR_ENOMEM;
  }
  if (s == EAR_OK && depth + 1 < REREDUCE_DEPTH && q->n_redges > 0)
    s = reduce_solve(p, q->n_reduced, q->n_redges, q->re_u, q->re_v, q->re_w, D, Np, comm, depth + 1, st, &inner,
                     levels, n_last);
  if (s == EAR_OK && !inner) {
    if (!comm) {
      if (by_sssp) {
        s = sssp_rows(q, D, Np, Np, 0, Np, nullptr, st);
      } else {
        s = fw_init_D(q, D, Np, Np, 0, Np, st);
        if (s == EAR_OK) s = fw_single(D, Np, Np, st, nullptr, q->n_reduced, allow16, q);   // connected
      }
    } else {
      const std::vector<int32_t> own = shard_rows(Np / TILE, P, comm->rank);
      int32_t *S = nullptr;   // the owned rows live in this rank's exchange window (read there by the gather)
      s = fw_shard_buffer(comm, Np, st, &S);
      if (by_sssp) {   // every rank its own tile rows, no exchange until the gather
        int32_t *d_rows = nullptr, nown = 0;
        if (s == EAR_OK) s = shard_rows_device(Np / TILE, P, comm->rank, &d_rows, &nown, st);
        if (s == EAR_OK) s = sssp_rows(q, S, Np, Np, 0, nown * TILE, d_rows, st);
        if (d_rows) cudaFreeAsync(d_rows, st);
      } else {
        for (size_t j = 0; j < own.size() && s == EAR_OK; ++j)
          s = fw_init_D(q, S + (int64_t)j * TILE * Np, Np, Np, own[j] * TILE, TILE, st);
        if (s == EAR_OK) s = fw_sharded_auto(S, Np, Np, comm, nullptr, q->n_reduced, allow16, st, q);
      }
      if (s == EAR_OK) s = fw_sharded_gather(S, Np, Np, D, Np, comm, st);
    }
  }
  if (s == EAR_OK) s = expand(q, D, Np, 0, n, M, ld, st, PK_REREDUCE);
  if (D) cudaFreeAsync(D, st);
  cudaStreamSynchronize(st);   // q's arrays are freed below
  plan_free(q);
  delete q;
  if (s == EAR_OK) *done = true;
  return s;
}

// The paper's order inside a big piece: its local edge list -> reduce_solve.
static ear_status_t piece_rereduce(ear_plan_s *p, ear_bcc_s *b, int32_t id, int32_t *M, int32_t ld, ear_comm_s *comm,
                                   cudaStream_t st, bool *done, int32_t *n_reduced) {
  *done = false;
  if (getenv("EAR_NO_REREDUCE")) return EAR_OK;   // development knob (A/B timing)
  const int32_t np = b->h_psize[id];
  const int32_t A = b->n_arcs;
  if (A <= 0) return EAR_OK;
  int32_t *e = nullptr;
  EAR_CUDA_TRY(cudaMallocAsync((void **)&e, sizeof(int32_t) * (3 * (size_t)A + 1), st));
  int32_t *cnt = e + 3 * (size_t)A;
  EAR_CUDA_TRY(dev_memset(cnt, 0, sizeof(int32_t), st));
  EAR_LAUNCH(k_piece_edges, grid_for(A), NT, 0, st)(b->arcs, A, id, e, e + A, e + 2 * (size_t)A, cnt);
  int32_t m = 0;
  {
    Readback rb(st);
    EAR_CUDA_TRY(rb.get(&m, cnt, sizeof(int32_t)));
    EAR_CUDA_TRY(rb.sync());
  }
  int32_t levels = 0, n_last = np;
  ear_status_t s = reduce_solve(p, np, m, e, e + A, e + 2 * (size_t)A, M, ld, comm, 0, st, done, &levels, &n_last);
  cudaFreeAsync(e, st);
  if (s == EAR_OK && *done) {
    *n_reduced = n_last;
    b->rereduced++;
    b->rereduce_levels = std::max(b->rereduce_levels, levels);
  }
  return s;
}

// Phase II by blocks: solve every piece, then compose rows of S^r into D.  Rows: [row0, row0 + rows)
// or, with d_tile_rows, the listed 128-row blocks (comm layout).  With a communicator the largest
// piece runs the sharded FW (its rows split over the ranks) and is re-assembled on every rank; the
// small pieces are solved redundantly.
ear_status_t bcc_solve(ear_plan_s *p, ear_comm_s *comm, int32_t *D, int64_t ldd, int32_t Np, int32_t row0,
                       int32_t rows, const int32_t *d_tile_rows, cudaStream_t st, uint16_t *D16, int64_t ld16,
                       int32_t *flag16) {
  NvtxRange nvtx_("ear: Phase II by blocks");
  const int32_t P = comm ? comm->nranks : 1;
  int sb = prof_begin(PK_BCC_PREP, st);
  ear_status_t sprep = bcc_prepare(p, P, st);
  prof_end(sb, st, 0);
  EAR_TRY(sprep);
  ear_bcc_s *b = p->bcc;
  const int32_t nr = p->n_reduced;
  EAR_CUDA_TRY(smem_attr((const void *)k_piece_fw, SMALL * SMALL * 4));
  int32_t *pool = nullptr;
  EAR_CUDA_TRY(cudaMallocAsync((void **)&pool, sizeof(int32_t) * (size_t)std::max<int64_t>(b->pool_ints, 4), st));
  ear_status_t s = EAR_OK;
  int sp = prof_begin(PK_BCC, st);
  EAR_LAUNCH(k_fill_pool, grid_for(b->pool_ints / 4 + 1), NT, 0, st)(pool, b->pool_ints);
  EAR_LAUNCH(k_pool_init, grid_for(std::max(nr, b->n_arcs)), NT, 0, st)(nr, b->cinfo, b->ridx, b->hp, b->pld,
                                                                         b->pbase, b->arcs, b->n_arcs, pool);
  if (b->n_pieces > 0)
    EAR_LAUNCH(k_piece_fw, b->n_pieces, NT, SMALL * SMALL * 4, st)(b->n_pieces, b->psize, b->pld, b->pbase, pool);
  prof_end(sp, st, 0);
  b->rereduced = 0;
  b->rereduce_levels = 0;
  b->largest_reduced = b->big.empty() ? b->largest : 0;
  for (size_t i = 0; i < b->big.size() && s == EAR_OK; ++i) {
    const int32_t id = b->big[i];
    int32_t *M = pool + b->h_pbase[id];
    const int32_t ld = b->h_pld[id];
    bool done = false;
    int32_t nred = b->h_psize[id];
    s = piece_rereduce(p, b, id, M, ld, (comm && i == 0) ? comm : nullptr, st, &done, &nred);
    if (i == 0) b->largest_reduced = nred;
    if (s != EAR_OK || done) continue;
    if (comm && i == 0) {   // the largest piece: sharded over the ranks, then gathered everywhere
      const int32_t nt = ld / TILE;
      std::vector<int32_t> own = shard_rows(nt, P, comm->rank);
      int32_t *S = nullptr;   // the owned rows live in this rank's exchange window (read there by the gather)
      s = fw_shard_buffer(comm, ld, st, &S);
      for (size_t j = 0; j < own.size() && s == EAR_OK; ++j)
        if (cudaMemcpyAsync(S + (int64_t)j * TILE * ld, M + (int64_t)own[j] * TILE * ld,
                            sizeof(int32_t) * (size_t)TILE * ld, cudaMemcpyDeviceToDevice, st) != cudaSuccess)
          s = EAR_ECUDA;
      if (s == EAR_OK)   // a piece is connected: no labels
        s = fw_sharded_auto(S, ld, ld, comm, nullptr, b->h_psize[id], !(p->flags & EAR_FLAG_FW32), st);
      if (s == EAR_OK) s = fw_sharded_gather(S, ld, ld, M, ld, comm, st);
    } else {
      s = fw_single(M, ld, ld, st, nullptr, b->h_psize[id], !(p->flags & EAR_FLAG_FW32));   // a piece is connected
    }
  }
  if (s == EAR_OK) {
    int sc = prof_begin(PK_COMPOSE, st);
    EAR_LAUNCH(k_hang_dist, grid_for(nr), NT, 0, st)(nr, b->att, b->hp, b->pld, b->pbase, pool, b->cinfo);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(rows, RB), 148 * 8));
    if (rows > 0)
      EAR_LAUNCH(k_compose, grid, NT, 0, st)(nr, Np, b->cinfo, b->hp, b->pld, b->pbase, pool, D, ldd, row0, rows,
                                             d_tile_rows, D16, ld16, flag16);
    prof_end(sc, st, (D ? 4.0 : 0.0) * rows * Np + (D16 ? 2.0 * rows * ld16 : 0.0));
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
      set_error("bcc_solve: %s", cudaGetErrorString(e));
      s = EAR_ECUDA;
    }
  }
  cudaFreeAsync(pool, st);
  return s;
}

}  // namespace ear

using namespace ear;

extern "C" ear_status_t ear_bcc_info(ear_plan_t p, ear_bcc_info_t *info) {
  if (!p || !info) {
    set_error("ear_bcc_info: NULL argument");
    return EAR_EINVAL;
  }
  EAR_TRY(bcc_prepare(p, p->bcc ? p->bcc->P : 1, p->stream));
  const ear_bcc_s *b = p->bcc;
  info->n_components = b->n_components;
  info->n_blocks = b->n_blocks;
  info->n_articulation = b->n_articulation;
  info->n_pieces = b->n_pieces;
  info->largest_piece = b->largest;
  info->tree_levels = b->levels;
  info->sum_cubes = b->sum_cubes;
  info->rereduced_pieces = b->rereduced;
  info->largest_reduced = b->largest_reduced;
  info->rereduce_levels = b->rereduce_levels;
  return EAR_OK;
}
