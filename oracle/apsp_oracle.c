/*
 * oracle/apsp_oracle.c -- CPU ORACLE. TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may load
 * this library.  The product path (paper_conf_ipps_duttackb17_b200/) never links, imports or calls
 * it, and it shares no code, header, table or helper with csrc/.
 *
 * What it computes (paper = /root/reference/PAPER.md, "P:NN" = line NN):
 *
 *  oracle_apsp_rows   S[s,t] = weight of a shortest s-t path in the ORIGINAL, uncontracted,
 *                     undirected graph G (P:41 problem statement, P:109 definition of S), computed
 *                     by Dijkstra's algorithm [9] from every requested source -- the paper's own SSSP
 *                     primitive (sec. 2.1.2) -- with a binary heap and int64 distances.
 *                     Unreachable -> ORACLE_INF (0x3FFFFFFF, reading C11); S[s,s] = 0.
 *                     Self-loops and parallel edges are simply relaxed like any other edge (a walk
 *                     never profits from a self-loop; the lighter parallel edge wins by itself).
 *                     Pins: tests/test_oracle_pins.py (brute-force FW on tiny graphs, exhaustive
 *                     enumeration, closed forms, scipy, invariants, Bellman certificate).
 *
 *  oracle_reduce      G^r = Reduce(G) as defined in P:88 (sec. 2.1.1) with the parallel-edge rule
 *                     of P:90, read for general graphs as in DESIGN.md readings C3-C7:
 *                       - self-loops dropped, parallel edges -> min weight, degree = #distinct nbrs;
 *                       - V^r = vertices of degree != 2 (C4), plus the minimum-id vertex of every
 *                         component that is a pure cycle (C5);
 *                       - every maximal chain of degree-2 vertices between two V^r vertices a, b
 *                         (a == b allowed: a closed ear, C6) becomes one G^r edge of weight
 *                         "the sum of the weights of the edges v x1, x1 x2, ..., xi w";
 *                       - for every chain vertex x: its two chain ends (left/right) and the
 *                         along-chain distance to each (reading C7 of wt(x, l_x)).
 *                     The walk is plain sequential code in the order the definition reads.
 *                     Pins: Fig. 4 chains, the cyclomatic identity of Lemma 3.1's proof
 *                      and brute-force checks in tests/test_oracle_pins.py.
 *
 *  oracle_certify_rows  a CHECKER, not a solver: whether candidate rows of S satisfy the Bellman
 *                     optimality equations of shortest paths in the ORIGINAL graph -- the definition
 *                     of S restated as a fixed point (SURVEY 8.c pin P4):
 *                       D[s][s] = 0;  D[s][t] = min over arcs (u,t) of D[s][u] + w(u,t)  (t != s),
 *                       ORACLE_INF when no u has a finite D[s][u].
 *                     With integer weights >= 1 the true distances are its ONLY solution: an entry
 *                     satisfying it is at most the weight of any s-t path (induction along the path),
 *                     and a finite entry is the weight of the walk spelled out by its strictly
 *                     decreasing chain of tight predecessors, which can only end at s.  O(N + M) per
 *                     row instead of Dijkstra's O(M log N): it certifies whole N x N matrices (cfg4,
 *                     cfg5) in seconds.  Pins: tests/test_oracle_pins.py (accepts the oracle's rows,
 *                     rejects every single-entry perturbation, exhaustive small graphs).
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC -o oracle/liboracle.so oracle/apsp_oracle.c
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_INF 0x3FFFFFFF

/* ------------------------------------------------------------------ adjacency (both directions) */
typedef struct {
  int32_t n;
  int64_t *start; /* n+1 */
  int32_t *nbr;   /* 2m */
  int64_t *wt;    /* 2m */
} adj_t;

static int adj_build(adj_t *g, int32_t n, int64_t m, const int32_t *src, const int32_t *dst,
                     const int32_t *w) {
  g->n = n;
  g->start = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  g->nbr = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * m + 1));
  g->wt = (int64_t *)malloc(sizeof(int64_t) * (size_t)(2 * m + 1));
  if (!g->start || !g->nbr || !g->wt) return -2;
  for (int64_t e = 0; e < m; ++e) {
    g->start[src[e] + 1]++;
    g->start[dst[e] + 1]++;
  }
  for (int32_t v = 0; v < n; ++v) g->start[v + 1] += g->start[v];
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  if (!fill) return -2;
  memcpy(fill, g->start, sizeof(int64_t) * (size_t)n);
  for (int64_t e = 0; e < m; ++e) {
    int32_t u = src[e], v = dst[e];
    g->nbr[fill[u]] = v; g->wt[fill[u]++] = w[e];
    g->nbr[fill[v]] = u; g->wt[fill[v]++] = w[e];
  }
  free(fill);
  return 0;
}

static void adj_free(adj_t *g) {
  free(g->start); free(g->nbr); free(g->wt);
}

static int validate(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w) {
  if (n < 1 || m < 0) return -1;
  for (int64_t e = 0; e < m; ++e) {
    if (src[e] < 0 || src[e] >= n || dst[e] < 0 || dst[e] >= n) return -1;
    if (w[e] < 1) return -1; /* W: E -> R+ (P:222); integer weights >= 1 (reading C1) */
  }
  return 0;
}

/* ------------------------------------------------------------------ Dijkstra, binary heap */
typedef struct { int64_t d; int32_t v; } item_t;

static void heap_push(item_t *h, int64_t *sz, item_t x) {
  int64_t i = (*sz)++;
  while (i > 0) {
    int64_t p = (i - 1) / 2;
    if (h[p].d <= x.d) break;
    h[i] = h[p]; i = p;
  }
  h[i] = x;
}

static item_t heap_pop(item_t *h, int64_t *sz) {
  item_t top = h[0], x = h[--(*sz)];
  int64_t i = 0;
  for (;;) {
    int64_t c = 2 * i + 1;
    if (c >= *sz) break;
    if (c + 1 < *sz && h[c + 1].d < h[c].d) c++;
    if (h[c].d >= x.d) break;
    h[i] = h[c]; i = c;
  }
  if (*sz > 0) h[i] = x;
  return top;
}

/* One source: dist[] (int64, -1 = unreached), lazy-deletion heap of capacity 2m + 1. */
static void dijkstra(const adj_t *g, int32_t s, int64_t *dist, item_t *heap) {
  int64_t sz = 0;
  for (int32_t v = 0; v < g->n; ++v) dist[v] = -1;
  dist[s] = 0;
  item_t it = {0, s};
  heap_push(heap, &sz, it);
  while (sz > 0) {
    item_t x = heap_pop(heap, &sz);
    if (x.d != dist[x.v]) continue; /* stale entry */
    for (int64_t k = g->start[x.v]; k < g->start[x.v + 1]; ++k) {
      int32_t y = g->nbr[k];
      int64_t nd = x.d + g->wt[k];
      if (dist[y] < 0 || nd < dist[y]) {
        dist[y] = nd;
        item_t z = {nd, y};
        heap_push(heap, &sz, z);
      }
    }
  }
}

/* Rows rows[0..nrows) of S, written to out[r * n + t] as int32 (unreachable -> ORACLE_INF).
 * Returns 0, -1 on invalid input, -2 on allocation failure, -5 if a finite distance >= INF. */
int oracle_apsp_rows(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w,
                     int32_t nrows, const int32_t *rows, int32_t *out, int32_t nthreads) {
  if (validate(n, m, src, dst, w)) return -1;
  for (int32_t r = 0; r < nrows; ++r)
    if (rows[r] < 0 || rows[r] >= n) return -1;
  adj_t g;
  if (adj_build(&g, n, m, src, dst, w)) { adj_free(&g); return -2; }
  int status = 0;
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
#pragma omp parallel
  {
    int64_t *dist = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    item_t *heap = (item_t *)malloc(sizeof(item_t) * (size_t)(2 * m + 2));
    if (!dist || !heap) {
#pragma omp atomic write
      status = -2;
    } else {
#pragma omp for schedule(dynamic, 1)
      for (int32_t r = 0; r < nrows; ++r) {
        dijkstra(&g, rows[r], dist, heap);
        int32_t *row = out + (int64_t)r * n;
        for (int32_t t = 0; t < n; ++t) {
          if (dist[t] < 0) row[t] = ORACLE_INF;
          else if (dist[t] >= ORACLE_INF) { row[t] = ORACLE_INF;
#pragma omp atomic write
            status = -5; }
          else row[t] = (int32_t)dist[t];
        }
      }
    }
    free(dist); free(heap);
  }
  adj_free(&g);
  return status;
}

/* Number of OpenMP threads a parallel region would use (for the reported core count). */
int oracle_num_threads(int32_t nthreads) {
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
  int t = 1;
#pragma omp parallel
  {
#pragma omp single
    t = omp_get_num_threads();
  }
  return t;
#else
  (void)nthreads;
  return 1;
#endif
}

/* ------------------------------------------------------------------ Reduce(G) */
/* Simple graph: sorted distinct neighbour lists with min weight, self-loops dropped (C3). */
typedef struct { int32_t v; int64_t w; } nb_t;

static int cmp_nb(const void *a, const void *b) {
  const nb_t *x = (const nb_t *)a, *y = (const nb_t *)b;
  if (x->v != y->v) return x->v < y->v ? -1 : 1;
  return (x->w > y->w) - (x->w < y->w);
}

/*
 * Outputs (caller-allocated):
 *   deg[n]        number of distinct neighbours (after C3)
 *   term[n]       1 if the vertex is in V^r
 *   end0[n], end1[n]   chain vertices: the two chain ends (vertex ids, end0 == end1 for a closed
 *                 ear); V^r vertices: end0 = end1 = itself
 *   d0[n], d1[n]  along-chain distance from the vertex to end0 / end1 (0 for V^r vertices)
 *   chain[n]      chain index of a chain vertex (0..n_chains-1), -1 for V^r vertices
 *   re_u, re_v, re_w  [cap] the G^r edge list BEFORE the parallel-edge rule: one entry per chain
 *                 (closed ears included as self-loops a == a) and one per direct V^r-V^r edge
 *   counts[0] = |V^r|, counts[1] = number of G^r edges written, counts[2] = number of chains,
 *   counts[3] = number of promoted pure-cycle anchors (C5)
 * Returns 0, -1 invalid input, -2 allocation failure, -3 if cap is too small.
 */
int oracle_reduce(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w,
                  int32_t *deg, int32_t *term, int32_t *end0, int32_t *end1, int64_t *d0, int64_t *d1,
                  int32_t *chain, int32_t *re_u, int32_t *re_v, int64_t *re_w, int64_t cap,
                  int64_t *counts) {
  if (validate(n, m, src, dst, w)) return -1;
  /* 1. simple graph (C3) */
  adj_t g;
  if (adj_build(&g, n, m, src, dst, w)) { adj_free(&g); return -2; }
  int64_t *s_start = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  nb_t *s_nb = (nb_t *)malloc(sizeof(nb_t) * (size_t)(2 * m + 1));
  if (!s_start || !s_nb) return -2;
  int64_t pos = 0;
  nb_t *tmp = (nb_t *)malloc(sizeof(nb_t) * (size_t)(2 * m + 1));
  for (int32_t v = 0; v < n; ++v) {
    int64_t k0 = g.start[v], k1 = g.start[v + 1], cnt = 0;
    for (int64_t k = k0; k < k1; ++k)
      if (g.nbr[k] != v) { tmp[cnt].v = g.nbr[k]; tmp[cnt].w = g.wt[k]; cnt++; }
    qsort(tmp, (size_t)cnt, sizeof(nb_t), cmp_nb);
    s_start[v] = pos;
    for (int64_t k = 0; k < cnt; ++k)
      if (k == 0 || tmp[k].v != tmp[k - 1].v) s_nb[pos++] = tmp[k]; /* first = min weight */
  }
  s_start[n] = pos;
  free(tmp);
  adj_free(&g);

  /* 2. degrees and V^r (C4) */
  for (int32_t v = 0; v < n; ++v) {
    deg[v] = (int32_t)(s_start[v + 1] - s_start[v]);
    term[v] = deg[v] != 2;
    chain[v] = -1;
    end0[v] = end1[v] = v;
    d0[v] = d1[v] = 0;
  }
  /* 3. pure cycles (C5): a component whose vertices all have degree 2; promote its min id.
   *    Walk each unvisited degree-2 vertex's component by plain traversal. */
  int32_t *comp_seen = (int32_t *)calloc((size_t)n, sizeof(int32_t));
  int32_t *stack = (int32_t *)malloc(sizeof(int32_t) * (size_t)n + 1);
  int64_t promoted = 0;
  for (int32_t v = 0; v < n; ++v) {
    if (comp_seen[v]) continue;
    int32_t sp = 0, minid = v, all2 = 1;
    stack[sp++] = v; comp_seen[v] = 1;
    while (sp > 0) {
      int32_t x = stack[--sp];
      if (deg[x] != 2) all2 = 0;
      if (x < minid) minid = x;
      for (int64_t k = s_start[x]; k < s_start[x + 1]; ++k) {
        int32_t y = s_nb[k].v;
        if (!comp_seen[y]) { comp_seen[y] = 1; stack[sp++] = y; }
      }
    }
    if (all2) { term[minid] = 1; promoted++; }
  }
  free(comp_seen); free(stack);

  /* 4. walk every chain from each of its V^r ends: from V^r vertex a through neighbour v,
   *    follow degree-2 vertices until the next V^r vertex b.  Each chain is walked from both ends;
   *    it is recorded (chain id, G^r edge) only on the walk whose first chain vertex was not yet
   *    visited.  Direct V^r-V^r edges are recorded once (a < b). */
  int64_t nre = 0, nchains = 0, nterm = 0;
  int32_t *path = (int32_t *)malloc(sizeof(int32_t) * (size_t)n + 1);
  int64_t *pre = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 2));
  int status = 0;
  for (int32_t a = 0; a < n; ++a) {
    if (!term[a]) continue;
    nterm++;
    for (int64_t k = s_start[a]; k < s_start[a + 1]; ++k) {
      int32_t v = s_nb[k].v;
      int64_t wsum = s_nb[k].w;
      if (term[v]) {
        if (a < v) {
          if (nre >= cap) { status = -3; goto done; }
          re_u[nre] = a; re_v[nre] = v; re_w[nre] = wsum; nre++;
        }
        continue;
      }
      if (chain[v] >= 0) continue; /* this chain was already walked from its other end */
      /* walk a -> v -> ... -> b */
      int32_t len = 0, prev = a, cur = v;
      pre[0] = wsum; /* pre[i] = distance from a to path[i] */
      while (!term[cur]) {
        path[len] = cur;
        /* next = the neighbour of cur other than prev (cur has exactly two distinct nbrs) */
        int64_t k0 = s_start[cur];
        int32_t nxt; int64_t wn;
        if (s_nb[k0].v != prev) { nxt = s_nb[k0].v; wn = s_nb[k0].w; }
        else { nxt = s_nb[k0 + 1].v; wn = s_nb[k0 + 1].w; }
        len++;
        pre[len] = pre[len - 1] + wn; /* distance from a to nxt */
        prev = cur; cur = nxt;
      }
      int32_t b = cur;
      int64_t L = pre[len];
      int32_t cid = (int32_t)nchains++;
      for (int32_t i = 0; i < len; ++i) {
        int32_t x = path[i];
        chain[x] = cid;
        end0[x] = a; d0[x] = pre[i];
        end1[x] = b; d1[x] = L - pre[i];
      }
      if (nre >= cap) { status = -3; goto done; }
      re_u[nre] = a; re_v[nre] = b; re_w[nre] = L; nre++;
    }
  }
done:
  counts[0] = nterm; counts[1] = nre; counts[2] = nchains; counts[3] = promoted;
  free(path); free(pre); free(s_start); free(s_nb);
  return status;
}

/* ------------------------------------------------------------------ Bellman certificate (checker)
 * Rows i < nrows of D (leading dimension ldd) are candidate rows S[rows[i], :].  Returns the number of
 * entries that violate the equations in the header (0: every row is exactly S), or a negative status;
 * first[0..1] = (i, t) of the first violation found (by row index); row_bad (may be NULL) gets the
 * violations of every row.  */
int64_t oracle_certify_rows(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w,
                            int32_t nrows, const int32_t *rows, const int32_t *D, int64_t ldd, int32_t nthreads,
                            int64_t *first, int64_t *row_bad_out) {
  if (validate(n, m, src, dst, w)) return -1;
  for (int32_t r = 0; r < nrows; ++r)
    if (rows[r] < 0 || rows[r] >= n) return -1;
  if (ldd < n) return -1;
  adj_t g;
  if (adj_build(&g, n, m, src, dst, w)) { adj_free(&g); return -2; }
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#endif
  int64_t bad = 0;
  first[0] = -1;
  first[1] = -1;
#pragma omp parallel for schedule(dynamic, 4) reduction(+ : bad)
  for (int32_t i = 0; i < nrows; ++i) {
    const int32_t s = rows[i];
    const int32_t *d = D + (int64_t)i * ldd;
    int64_t row_bad = 0;
    int32_t first_t = -1;
    for (int32_t t = 0; t < n; ++t) {
      int64_t expect;
      if (t == s) {
        expect = 0;
      } else {
        int64_t best = ORACLE_INF;   /* min over the arcs (u, t); the graph is undirected */
        for (int64_t a = g.start[t]; a < g.start[t + 1]; ++a) {
          const int32_t u = g.nbr[a];
          const int64_t du = d[u];
          if (u == t || du < 0 || du >= ORACLE_INF) continue;   /* self-loop, or no finite path to u */
          if (du + g.wt[a] < best) best = du + g.wt[a];
        }
        expect = best;
      }
      if ((int64_t)d[t] != expect) {
        if (first_t < 0) first_t = t;
        ++row_bad;
      }
    }
    if (row_bad_out) row_bad_out[i] = row_bad;
    if (row_bad) {
#pragma omp critical
      {
        if (first[0] < 0 || i < first[0]) { first[0] = i; first[1] = first_t; }
      }
      bad += row_bad;
    }
  }
  adj_free(&g);
  return bad;
}
