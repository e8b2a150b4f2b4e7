// Phase I -- G^r = Reduce(G) (Alg. 1 line 2; definition; parallel-edge rule P:90).
//
// Data-parallel chain contraction:
//   a1  canonicalise: arcs (u,v) of both directions, self-loops dropped, sorted by (u,v) and
//       reduced by key with min weight -> symmetric CSR of the simple graph (reading C3);
//   a2  degree = #distinct neighbours; terminal = degree != 2 (C4) (all vertices with
//       EAR_FLAG_NO_CONTRACT);
//   a3  chain ranking by pointer jumping (Wyllie list ranking) over ARCS: an arc u->v whose head v
//       has degree two continues with v->x (x != u).  ceil(log2 Lmax) synchronous doubling rounds
//       give every arc the terminal it reaches, the distance to it and the last arc entering it.
//       A round that finishes no arc while arcs remain active proves the remaining arcs lie on
//       pure cycles (C5): a min-label doubling pass finds the minimum vertex id of each such
//       cycle, which is promoted to a terminal, and the ranking is redone;
//   a4  terminal ids by exclusive scan (monotone in caller id), per-vertex descriptors
//       {tid(left), d(left), tid(right), d(right)} with left = the end with the smaller
//       (end id, entering-arc id) and chain id = the smaller entering-arc id (reading C8), the
//       reduced arcs (tail terminal -> end terminal, chain weight sum; closed ears dropped,
//       C6), and the same-chain vertex lists for the along-chain rule.
#include <cub/cub.cuh>

#include <algorithm>
#include <vector>

#include "common.cuh"

namespace ear {
namespace {

constexpr int NT = 256;

inline int grid_for(int64_t n) { return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, NT), 1 << 20)); }

#define GRID_STRIDE(i, n) for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (n); i += (int64_t)gridDim.x * blockDim.x)

// ------------------------------------------------------------------------------------- a1
__global__ void k_validate(const int32_t *src, const int32_t *dst, const int32_t *w, int64_t m, int32_t n,
                           int32_t *flags /* [0]=bad, [1]=wmax, [2]=self-loops */) {
  int bad = 0, wmax = 0, loops = 0;
  GRID_STRIDE(i, m) {
    int32_t u = src[i], v = dst[i], x = w[i];
    if (u < 0 || u >= n || v < 0 || v >= n || x < 1) bad = 1;
    wmax = max(wmax, x);
    loops += (u == v);
  }
  if (bad) atomicOr(&flags[0], 1);
  atomicMax(&flags[1], wmax);
  if (loops) atomicAdd(&flags[2], loops);
}

// both directions of every edge; self-loops get the sentinel key (sorted past every real arc)
__global__ void k_make_arcs(const int32_t *src, const int32_t *dst, const int32_t *w, int64_t m,
                            uint64_t sentinel, uint64_t *keys, int32_t *vals) {
  GRID_STRIDE(i, m) {
    uint32_t u = (uint32_t)src[i], v = (uint32_t)dst[i];
    bool loop = u == v;
    keys[2 * i] = loop ? sentinel : ((uint64_t)u << 32 | v);
    keys[2 * i + 1] = loop ? sentinel : ((uint64_t)v << 32 | u);
    vals[2 * i] = w[i];
    vals[2 * i + 1] = w[i];
  }
}

struct MinOp {
  __device__ __forceinline__ int32_t operator()(int32_t a, int32_t b) const { return a < b ? a : b; }
};

__global__ void k_split_arcs(const uint64_t *keys, int64_t A, int32_t *asrc, int32_t *adst, int32_t *deg) {
  GRID_STRIDE(a, A) {
    uint64_t k = keys[a];
    int32_t u = (int32_t)(k >> 32), v = (int32_t)(k & 0xFFFFFFFFu);
    asrc[a] = u;
    adst[a] = v;
    atomicAdd(&deg[u], 1);
  }
}

// ------------------------------------------------------------------------------------- a2
__global__ void k_terminals(const int32_t *deg, int32_t n, uint32_t flags, int32_t *term) {
  GRID_STRIDE(v, n) { term[v] = (flags & EAR_FLAG_NO_CONTRACT) ? 1 : (deg[v] != 2); }
}

// ------------------------------------------------------------------------------------- a3
// successor arc of a (head v of degree two): the arc out of v that does not return to tail(a)
__device__ __forceinline__ int32_t succ_arc(int32_t a, const int32_t *asrc, const int32_t *adst,
                                            const int32_t *rowptr) {
  int32_t v = adst[a];
  int32_t r = rowptr[v];
  return adst[r] == asrc[a] ? r + 1 : r;
}

struct RankBuf {
  int32_t *nxt, *end, *last;
  uint32_t *sum;
  uint8_t *done;
};

__global__ void k_rank_init(int64_t A, const int32_t *asrc, const int32_t *adst, const int32_t *aw,
                            const int32_t *rowptr, const int32_t *term, RankBuf b) {
  GRID_STRIDE(a, A) {
    int32_t v = adst[a];
    b.sum[a] = (uint32_t)aw[a];
    if (term[v]) {
      b.done[a] = 1; b.end[a] = v; b.last[a] = (int32_t)a; b.nxt[a] = -1;
    } else {
      b.done[a] = 0; b.end[a] = -1; b.last[a] = -1;
      b.nxt[a] = succ_arc((int32_t)a, asrc, adst, rowptr);
    }
  }
}

// One synchronous Wyllie doubling round (double-buffered: reads `in`, writes `out`).
// counters[0] += arcs finished this round, counters[1] += arcs still active after it.
__global__ void k_rank_round(int64_t A, RankBuf in, RankBuf out, unsigned long long *counters) {
  unsigned fin = 0, act = 0;
  GRID_STRIDE(a, A) {
    if (in.done[a]) {
      out.done[a] = 1; out.end[a] = in.end[a]; out.last[a] = in.last[a]; out.sum[a] = in.sum[a];
      out.nxt[a] = -1;
    } else {
      int32_t nx = in.nxt[a];
      out.sum[a] = in.sum[a] + in.sum[nx];   // unsigned: pure-cycle arcs may wrap; discarded later
      if (in.done[nx]) {
        out.done[a] = 1; out.end[a] = in.end[nx]; out.last[a] = in.last[nx]; out.nxt[a] = -1;
        fin++;
      } else {
        out.done[a] = 0; out.end[a] = -1; out.last[a] = -1; out.nxt[a] = in.nxt[nx];
        act++;
      }
    }
  }
  // warp-aggregate the counters
  for (int o = 16; o > 0; o >>= 1) {
    fin += __shfl_down_sync(0xffffffffu, fin, o);
    act += __shfl_down_sync(0xffffffffu, act, o);
  }
  if ((threadIdx.x & 31) == 0) {
    if (fin) atomicAdd(&counters[0], (unsigned long long)fin);
    if (act) atomicAdd(&counters[1], (unsigned long long)act);
  }
}

// pure cycles (C5): min tail id along each cycle by doubling
__global__ void k_cycle_init(int64_t A, const uint8_t *done, const int32_t *asrc, const int32_t *adst,
                             const int32_t *rowptr, int32_t *lab, int32_t *nxt) {
  GRID_STRIDE(a, A) {
    if (!done[a]) {
      lab[a] = asrc[a];
      nxt[a] = succ_arc((int32_t)a, asrc, adst, rowptr);
    }
  }
}

__global__ void k_cycle_round(int64_t A, const uint8_t *done, const int32_t *lab_in, const int32_t *nxt_in,
                              int32_t *lab_out, int32_t *nxt_out, int32_t *changed) {
  int ch = 0;
  GRID_STRIDE(a, A) {
    if (!done[a]) {
      int32_t nx = nxt_in[a];
      int32_t l = min(lab_in[a], lab_in[nx]);
      ch |= (l != lab_in[a]);
      lab_out[a] = l;
      nxt_out[a] = nxt_in[nx];
    }
  }
  if (__any_sync(0xffffffffu, ch) && (threadIdx.x & 31) == 0) atomicOr(changed, 1);
}

__global__ void k_cycle_promote(int64_t A, const uint8_t *done, const int32_t *asrc, const int32_t *lab,
                                int32_t *term) {
  GRID_STRIDE(a, A) {
    if (!done[a] && asrc[a] == lab[a]) term[asrc[a]] = 1;
  }
}

// ------------------------------------------------------------------------------------- a4
__global__ void k_descriptors(int32_t n, const int32_t *term, const int32_t *scan, const int32_t *rowptr,
                              RankBuf b, VDesc *desc, int32_t *tid, int32_t *ear, int32_t *ear_cnt,
                              uint64_t *seg_key, int32_t *seg_val, uint64_t seg_sentinel) {
  GRID_STRIDE(v, n) {
    if (term[v]) {
      int32_t t = scan[v];
      desc[v] = VDesc{t, 0, t, 0};
      tid[v] = t;
      ear[v] = -1;
      seg_key[v] = seg_sentinel;
    } else {
      int32_t a1 = rowptr[v], a2 = a1 + 1;
      int32_t e1 = b.end[a1], l1 = b.last[a1], e2 = b.end[a2], l2 = b.last[a2];
      int32_t d1 = (int32_t)b.sum[a1], d2 = (int32_t)b.sum[a2];
      bool first_is_left = (e1 < e2) || (e1 == e2 && l1 < l2);
      int32_t el = first_is_left ? e1 : e2, dl = first_is_left ? d1 : d2;
      int32_t er = first_is_left ? e2 : e1, dr = first_is_left ? d2 : d1;
      int32_t id = min(l1, l2);
      desc[v] = VDesc{scan[el], dl, scan[er], dr};
      tid[v] = -1;
      ear[v] = id;
      atomicAdd(&ear_cnt[id], 1);
      seg_key[v] = ((uint64_t)(uint32_t)id << 32) | (uint32_t)dl;
    }
    seg_val[v] = (int32_t)v;
  }
}

__global__ void k_chain_stats(int64_t A, const int32_t *ear_cnt, int32_t *stats /* [0]=chains [1]=max */) {
  int c = 0, mx = 0;
  GRID_STRIDE(a, A) {
    int32_t k = ear_cnt[a];
    c += k > 0;
    mx = max(mx, k);
  }
  for (int o = 16; o > 0; o >>= 1) {
    c += __shfl_down_sync(0xffffffffu, c, o);
    mx = max(mx, __shfl_down_sync(0xffffffffu, mx, o));
  }
  if ((threadIdx.x & 31) == 0) {
    if (c) atomicAdd(&stats[0], c);
    atomicMax(&stats[1], mx);
  }
}

// segments of the sorted (chain id, offset) list: head flags
__global__ void k_seg_heads(int32_t nc, const uint64_t *keys, int32_t *head) {
  GRID_STRIDE(i, nc) { head[i] = (i == 0) || ((keys[i] >> 32) != (keys[i - 1] >> 32)); }
}

__global__ void k_seg_fill(int32_t nc, const int32_t *head, const int32_t *segscan, const int32_t *verts,
                           int32_t *seg_start, int32_t *seg_of, int32_t *seg_vert) {
  GRID_STRIDE(i, nc) {
    int32_t s = segscan[i] - 1;   // inclusive scan of heads
    if (head[i]) seg_start[s] = (int32_t)i;
    seg_of[verts[i]] = s;
    seg_vert[i] = verts[i];
  }
}

__global__ void k_seg_last(int32_t nseg, int32_t nc, int32_t *seg_start) { seg_start[nseg] = nc; }

// reduced arcs: tail terminal u, end terminal e != u (closed ears dropped, C6); rx: the first vertex
// after u (the chain's first interior vertex), or -1 when the arc is a direct terminal-terminal edge
__global__ void k_reduced_arcs(int64_t A, const int32_t *asrc, const int32_t *adst, const int32_t *term,
                               const int32_t *scan, RankBuf b, int32_t *ru, int32_t *rv, int32_t *rw, int32_t *rx,
                               unsigned long long *count, int emit) {
  GRID_STRIDE(a, A) {
    int32_t u = asrc[a];
    if (term[u]) {
      int32_t e = b.end[a];
      if (e != u) {
        unsigned long long k = atomicAdd(count, 1ull);
        if (emit) {
          ru[k] = scan[u];
          rv[k] = scan[e];
          rw[k] = (int32_t)b.sum[a];
          rx[k] = term[adst[a]] ? -1 : adst[a];
        }
      }
    }
  }
}

__global__ void k_count_promoted(int32_t n, const int32_t *deg, const int32_t *term, int32_t *out) {
  int c = 0;
  GRID_STRIDE(v, n) c += (term[v] && deg[v] == 2);
  for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(out, c);
}

__global__ void k_fill_neg(int32_t *p, int64_t n) {
  GRID_STRIDE(i, n) p[i] = -1;
}

int bitlen(uint64_t x) {
  int b = 0;
  while (x) { b++; x >>= 1; }
  return b;
}

// RAII-free scratch list: freed on every exit path of decompose
struct Scratch {
  cudaStream_t s;
  std::vector<void *> ptrs;
  template <class T>
  ear_status_t alloc(T **p, int64_t count) {
    *p = nullptr;
    if (count <= 0) count = 1;
    cudaError_t e = cudaMallocAsync((void **)p, sizeof(T) * (size_t)count, s);
    if (e != cudaSuccess) {
      set_error("cudaMallocAsync(%lld bytes): %s", (long long)(sizeof(T) * count), cudaGetErrorString(e));
      return EAR_ENOMEM;
    }
    ptrs.push_back(*p);
    return EAR_OK;
  }
  ~Scratch() {
    for (void *p : ptrs) cudaFreeAsync(p, s);
  }
};

}  // namespace

// Plan arrays come from the device's stream-ordered pool (cached; no driver call in steady state)
// and are released in stream order on the stream the plan was created on.
void plan_free(ear_plan_s *p) {
  if (!p) return;
  void *arrs[] = {p->desc, p->tid, p->ear, p->seg_of, p->seg_start, p->seg_vert, p->re_u, p->re_v, p->re_w, p->re_x,
                  p->r_rowptr, p->r_col, p->r_w, p->r_arcs, p->r_ell16, p->r_maxnb};
  for (void *a : arrs)
    if (a) cudaFreeAsync(a, p->stream);
  bcc_free(p->bcc, p->stream);
  p->bcc = nullptr;
  xp_free(p->xp, p->stream);
  p->xp = nullptr;
  part_free(p->part, p->stream);
  p->part = nullptr;
  if (p->cc) cudaFreeAsync(p->cc, p->stream);
  p->cc = nullptr;
}

template <class T>
static ear_status_t plan_alloc(T **p, int64_t count, cudaStream_t st) {
  if (count <= 0) count = 1;
  cudaError_t e = cudaMallocAsync((void **)p, sizeof(T) * (size_t)count, st);
  if (e != cudaSuccess) {
    set_error("cudaMallocAsync: %s", cudaGetErrorString(e));
    return EAR_ENOMEM;
  }
  return EAR_OK;
}

ear_status_t decompose(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w,
                       uint32_t flags, cudaStream_t st, ear_plan_s *plan) {
  plan->n = n;
  plan->flags = flags;
  plan->stream = st;
  Scratch S{st, {}};
  LabTrace tr(st, -5);

  // ---- validation (reads the flags back at the N_r synchronisation point below; an invalid input
  //      must not be processed further, so we sync once here as well -- cheap).
  int32_t *d_flags;
  EAR_TRY(S.alloc(&d_flags, 8));
  EAR_CUDA_TRY(dev_memset(d_flags, 0, sizeof(int32_t) * 8, st));
  if (m > 0) EAR_LAUNCH(k_validate, grid_for(m), NT, 0, st)(src, dst, w, m, n, d_flags);
  int32_t h_flags[3];
  {
    Readback rb(st);
    EAR_CUDA_TRY(rb.get(h_flags, d_flags, sizeof(h_flags)));
    EAR_CUDA_TRY(rb.sync());
  }
  if (h_flags[0]) {
    set_error("ear_decompose: vertex id out of [0,%d) or weight < 1", n);
    return EAR_EINVAL;
  }
  plan->max_weight = h_flags[1];
  if ((int64_t)(n - 1) * (int64_t)h_flags[1] >= (int64_t)INF) {
    set_error("ear_decompose: (n-1)*max weight = %lld >= EAR_INF", (long long)(n - 1) * h_flags[1]);
    return EAR_EOVERFLOW;
  }

  tr.mark("decompose: validate");
  // ---- a1: arcs, sort, reduce-by-key(min)
  const int64_t M2 = 2 * m;
  const uint64_t sentinel = (uint64_t)(uint32_t)n << 32;
  const int end_bit = 32 + bitlen((uint64_t)n);
  uint64_t *keys_a, *keys_b;
  int32_t *vals_a, *vals_b;
  EAR_TRY(S.alloc(&keys_a, M2)); EAR_TRY(S.alloc(&keys_b, M2));
  EAR_TRY(S.alloc(&vals_a, M2)); EAR_TRY(S.alloc(&vals_b, M2));
  if (m > 0) EAR_LAUNCH(k_make_arcs, grid_for(m), NT, 0, st)(src, dst, w, m, sentinel, keys_a, vals_a);

  uint64_t *ukeys;
  int32_t *uw, *d_nruns;
  EAR_TRY(S.alloc(&ukeys, M2)); EAR_TRY(S.alloc(&uw, M2)); EAR_TRY(S.alloc(&d_nruns, 1));
  int64_t A = 0;
  if (M2 > 0) {
    size_t tb_sort = 0, tb_red = 0;
    cub::DoubleBuffer<uint64_t> dk(keys_a, keys_b);
    cub::DoubleBuffer<int32_t> dv(vals_a, vals_b);
    cub::DeviceRadixSort::SortPairs(nullptr, tb_sort, dk, dv, (int)M2, 0, end_bit, st);
    cub::DeviceReduce::ReduceByKey(nullptr, tb_red, keys_a, ukeys, vals_a, uw, d_nruns, MinOp(), (int)M2, st);
    void *tmp;
    EAR_TRY(S.alloc((char **)&tmp, (int64_t)std::max(tb_sort, tb_red)));
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb_sort, dk, dv, (int)M2, 0, end_bit, st));
    EAR_CUDA_TRY(cub::DeviceReduce::ReduceByKey(tmp, tb_red, dk.Current(), ukeys, dv.Current(), uw, d_nruns,
                                                MinOp(), (int)M2, st));
    int32_t h_runs;
    Readback rbk(st);
    EAR_CUDA_TRY(rbk.get(&h_runs, d_nruns, sizeof(int32_t)));
    EAR_CUDA_TRY(rbk.sync());
    A = h_runs - (h_flags[2] > 0 ? 1 : 0);   // drop the self-loop sentinel run
  }
  plan->m_simple = A / 2;

  // CSR of the simple graph
  int32_t *asrc, *adst, *deg, *rowptr, *term, *scan;
  EAR_TRY(S.alloc(&asrc, A)); EAR_TRY(S.alloc(&adst, A));
  EAR_TRY(S.alloc(&deg, n + 1)); EAR_TRY(S.alloc(&rowptr, n + 1));
  EAR_TRY(S.alloc(&term, n)); EAR_TRY(S.alloc(&scan, n + 1));
  EAR_CUDA_TRY(dev_memset(deg, 0, sizeof(int32_t) * (n + 1), st));
  if (A > 0) EAR_LAUNCH(k_split_arcs, grid_for(A), NT, 0, st)(ukeys, A, asrc, adst, deg);
  {
    size_t tb = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tb, deg, rowptr, n + 1, st);
    void *tmp;
    EAR_TRY(S.alloc((char **)&tmp, (int64_t)tb));
    EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb, deg, rowptr, n + 1, st));
  }

  tr.mark("decompose: a1 sort/CSR");
  // ---- a2
  EAR_LAUNCH(k_terminals, grid_for(n), NT, 0, st)(deg, n, flags, term);

  // ---- a3: pointer-jumping chain ranking (ping-pong buffers)
  RankBuf rb[2];
  for (int i = 0; i < 2; ++i) {
    EAR_TRY(S.alloc(&rb[i].nxt, A)); EAR_TRY(S.alloc(&rb[i].end, A)); EAR_TRY(S.alloc(&rb[i].last, A));
    EAR_TRY(S.alloc(&rb[i].sum, A)); EAR_TRY(S.alloc(&rb[i].done, A));
  }
  unsigned long long *d_cnt;
  EAR_TRY(S.alloc(&d_cnt, 4));
  int cur = 0;
  int total_rounds = 0;
  plan->n_promoted = 0;
  for (int pass = 0; pass < 2; ++pass) {
    cur = 0;
    if (A > 0) EAR_LAUNCH(k_rank_init, grid_for(A), NT, 0, st)(A, asrc, adst, uw, rowptr, term, rb[0]);
    bool cycles = false;
    for (int round = 0; A > 0; ++round) {
      EAR_CUDA_TRY(dev_memset(d_cnt, 0, sizeof(unsigned long long) * 2, st));
      EAR_LAUNCH(k_rank_round, grid_for(A), NT, 0, st)(A, rb[cur], rb[cur ^ 1], d_cnt);
      cur ^= 1;
      total_rounds++;
      unsigned long long h_cnt[2];
      Readback rbk(st);
      EAR_CUDA_TRY(rbk.get(h_cnt, d_cnt, sizeof(h_cnt)));
      EAR_CUDA_TRY(rbk.sync());
      if (h_cnt[1] == 0) break;                      // every arc ranked
      if (h_cnt[0] == 0) { cycles = true; break; }   // only pure-cycle arcs remain (C5)
    }
    if (!cycles) break;
    if (pass == 1) {
      set_error("ear_decompose: chain ranking did not converge after pure-cycle promotion");
      return EAR_ECUDA;
    }
    // min-label doubling over the remaining (cycle) arcs, then promote the min-id vertex
    int32_t *lab[2], *cn[2], *d_changed;
    for (int i = 0; i < 2; ++i) { EAR_TRY(S.alloc(&lab[i], A)); EAR_TRY(S.alloc(&cn[i], A)); }
    EAR_TRY(S.alloc(&d_changed, 1));
    EAR_LAUNCH(k_cycle_init, grid_for(A), NT, 0, st)(A, rb[cur].done, asrc, adst, rowptr, lab[0], cn[0]);
    int c = 0;
    for (;;) {
      EAR_CUDA_TRY(dev_memset(d_changed, 0, sizeof(int32_t), st));
      EAR_LAUNCH(k_cycle_round, grid_for(A), NT, 0, st)(A, rb[cur].done, lab[c], cn[c], lab[c ^ 1], cn[c ^ 1], d_changed);
      c ^= 1;
      total_rounds++;
      int32_t h_changed;
      Readback rbk(st);
      EAR_CUDA_TRY(rbk.get(&h_changed, d_changed, sizeof(int32_t)));
      EAR_CUDA_TRY(rbk.sync());
      if (!h_changed) break;
    }
    EAR_LAUNCH(k_cycle_promote, grid_for(A), NT, 0, st)(A, rb[cur].done, asrc, lab[c], term);
    plan->n_promoted = -1;  // counted below
  }
  plan->rank_rounds = total_rounds;

  tr.mark("decompose: a2-a3 ranking");
  // ---- a4: terminal ids
  {
    size_t tb = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tb, term, scan, n, st);
    void *tmp;
    EAR_TRY(S.alloc((char **)&tmp, (int64_t)tb));
    EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb, term, scan, n, st));
  }
  int32_t h_last[2];
  Readback rbk(st);   // delivered at the N_r synchronisation point below
  EAR_CUDA_TRY(rbk.get(&h_last[0], scan + n - 1, sizeof(int32_t)));
  EAR_CUDA_TRY(rbk.get(&h_last[1], term + n - 1, sizeof(int32_t)));

  // descriptors
  EAR_TRY(plan_alloc(&plan->desc, n, st));
  EAR_TRY(plan_alloc(&plan->tid, n, st));
  EAR_TRY(plan_alloc(&plan->ear, n, st));
  EAR_TRY(plan_alloc(&plan->seg_of, n, st));
  int32_t *ear_cnt, *d_stats;
  uint64_t *seg_key, *seg_key2;
  int32_t *seg_val, *seg_val2;
  EAR_TRY(S.alloc(&ear_cnt, A)); EAR_TRY(S.alloc(&d_stats, 2));
  EAR_TRY(S.alloc(&seg_key, n)); EAR_TRY(S.alloc(&seg_key2, n));
  EAR_TRY(S.alloc(&seg_val, n)); EAR_TRY(S.alloc(&seg_val2, n));
  EAR_CUDA_TRY(dev_memset(ear_cnt, 0, sizeof(int32_t) * std::max<int64_t>(A, 1), st));
  EAR_CUDA_TRY(dev_memset(d_stats, 0, sizeof(int32_t) * 2, st));
  const uint64_t seg_sentinel = (uint64_t)(uint32_t)std::max<int64_t>(A, 1) << 32;
  EAR_LAUNCH(k_descriptors, grid_for(n), NT, 0, st)(n, term, scan, rowptr, rb[cur], plan->desc, plan->tid, plan->ear,
                                            ear_cnt, seg_key, seg_val, seg_sentinel);
  if (A > 0) EAR_LAUNCH(k_chain_stats, grid_for(A), NT, 0, st)(A, ear_cnt, d_stats);

  // reduced arcs: count, then emit
  unsigned long long *d_rcount;
  EAR_TRY(S.alloc(&d_rcount, 1));
  EAR_CUDA_TRY(dev_memset(d_rcount, 0, sizeof(unsigned long long), st));
  if (A > 0)
    EAR_LAUNCH(k_reduced_arcs, grid_for(A), NT, 0, st)(A, asrc, adst, term, scan, rb[cur], nullptr, nullptr, nullptr,
                                                       nullptr, d_rcount, 0);
  unsigned long long h_rcount = 0;
  int32_t h_stats[2];
  EAR_CUDA_TRY(rbk.get(&h_rcount, d_rcount, sizeof(h_rcount)));
  EAR_CUDA_TRY(rbk.get(h_stats, d_stats, sizeof(h_stats)));
  EAR_CUDA_TRY(rbk.sync());
  plan->n_reduced = h_last[0] + h_last[1];
  plan->n_chains = h_stats[0];
  plan->max_chain_len = h_stats[1];
  plan->n_redges = (int64_t)h_rcount;
  EAR_TRY(plan_alloc(&plan->re_u, plan->n_redges, st));
  EAR_TRY(plan_alloc(&plan->re_v, plan->n_redges, st));
  EAR_TRY(plan_alloc(&plan->re_w, plan->n_redges, st));
  EAR_TRY(plan_alloc(&plan->re_x, plan->n_redges, st));
  EAR_CUDA_TRY(dev_memset(d_rcount, 0, sizeof(unsigned long long), st));
  if (A > 0)
    EAR_LAUNCH(k_reduced_arcs, grid_for(A), NT, 0, st)(A, asrc, adst, term, scan, rb[cur], plan->re_u, plan->re_v,
                                                       plan->re_w, plan->re_x, d_rcount, 1);

  // same-chain vertex lists sorted by (chain id, off_left)
  const int32_t nc = n - plan->n_reduced;
  plan->n_chain_vertices = nc;
  EAR_TRY(plan_alloc(&plan->seg_start, (int64_t)plan->n_chains + 1, st));
  EAR_TRY(plan_alloc(&plan->seg_vert, nc, st));
  if (nc > 0) {
    size_t tb = 0;
    cub::DoubleBuffer<uint64_t> dk(seg_key, seg_key2);
    cub::DoubleBuffer<int32_t> dv(seg_val, seg_val2);
    const int kbits = 32 + bitlen((uint64_t)std::max<int64_t>(A, 1));
    cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, n, 0, kbits, st);
    void *tmp;
    EAR_TRY(S.alloc((char **)&tmp, (int64_t)tb));
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dv, n, 0, kbits, st));
    int32_t *head, *hscan;
    EAR_TRY(S.alloc(&head, nc)); EAR_TRY(S.alloc(&hscan, nc));
    EAR_LAUNCH(k_seg_heads, grid_for(nc), NT, 0, st)(nc, dk.Current(), head);
    size_t tb2 = 0;
    cub::DeviceScan::InclusiveSum(nullptr, tb2, head, hscan, nc, st);
    void *tmp2;
    EAR_TRY(S.alloc((char **)&tmp2, (int64_t)tb2));
    EAR_CUDA_TRY(cub::DeviceScan::InclusiveSum(tmp2, tb2, head, hscan, nc, st));
    EAR_LAUNCH(k_fill_neg, grid_for(n), NT, 0, st)(plan->seg_of, n);
    EAR_LAUNCH(k_seg_fill, grid_for(nc), NT, 0, st)(nc, head, hscan, dv.Current(), plan->seg_start, plan->seg_of,
                                            plan->seg_vert);
    EAR_LAUNCH(k_seg_last, 1, 1, 0, st)(plan->n_chains, nc, plan->seg_start);
  } else {
    EAR_LAUNCH(k_fill_neg, grid_for(n), NT, 0, st)(plan->seg_of, n);
    EAR_LAUNCH(k_seg_last, 1, 1, 0, st)(0, 0, plan->seg_start);
  }
  if (plan->n_promoted < 0) {
    // promoted pure-cycle anchors = terminals of degree two (C5)
    EAR_CUDA_TRY(dev_memset(d_stats, 0, sizeof(int32_t), st));
    EAR_LAUNCH(k_count_promoted, grid_for(n), NT, 0, st)(n, deg, term, d_stats);
    EAR_CUDA_TRY(rbk.get(h_stats, d_stats, sizeof(int32_t)));
  }
  EAR_CUDA_TRY(cudaGetLastError());
  EAR_CUDA_TRY(rbk.sync());
  if (plan->n_promoted < 0) plan->n_promoted = h_stats[0];
  tr.mark("decompose: a4 + chains");
  return EAR_OK;
}

}  // namespace ear
