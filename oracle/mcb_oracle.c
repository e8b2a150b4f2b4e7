/*
 * oracle/mcb_oracle.c -- CPU ORACLE for the minimum cycle basis (MCB).  TEST INFRASTRUCTURE ONLY
 * (same rules as apsp_oracle.c: only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg
 * may load it; nothing is shared with csrc/).
 *
 * Problem (paper sec. 3.1): an undirected multigraph G with weights W: E -> R+ (integers
 * >= 1 here, reading C1); its cycle space over GF(2) has dimension f = m - n + k (k components); an MCB
 * is a basis of it of minimum total weight.  Self-loops and parallel edges are allowed (the reduced
 * graph G^r "may contain multiple edges and self-loops"): a self-loop is a cycle by itself and
 * two parallel edges form a 2-cycle.  The MCB weight is unique; the basis need not be.
 *
 *  oracle_mcb_horton   Horton's algorithm [18]: for every vertex x a shortest-path tree
 *                      T_x (Dijkstra, int64); the Horton cycles C(x, e) = P_x(u) + e + P_x(v) for every
 *                      edge e = (u, v) not in T_x whose two tree paths meet only at x (self-loops at x:
 *                      the loop alone); sorted by weight; a GF(2) greedy keeps a cycle iff it is
 *                      independent of those kept (Gaussian elimination on edge-incidence bit vectors)
 *                      until f are kept.  Horton's theorem: the Horton set contains an MCB, and the
 *                      cycle-space matroid makes the greedy optimal.
 *  oracle_mcb_depina   de Pina's Algorithm 2 step by step: a spanning tree T (BFS), the
 *                      non-tree edges E' = {e_1..e_f} in edge order, witnesses S_i = unit vectors; in
 *                      phase i the shortest cycle C with <C, S_i> = 1 by the signed auxiliary graph of
 *                      sec. 3.2.1 (x+/x- per vertex, an edge keeps the sign unless it is in
 *                      the support of S_i -- reading M2 of DESIGN.md -- and a shortest x+ -> x- path is a
 *                      shortest cycle through x with odd S_i-parity), minimised over x; then every later
 *                      witness S_j with <C_i, S_j> = 1 becomes S_j xor S_i (lines 4-8).  O(f n m log n):
 *                      small graphs only, a second, independent route to the same weight.
 * Pins: tests/test_oracle_pins.py (brute force over the whole cycle space of tiny graphs, closed forms
 * for cycles, grids, theta graphs, K4 and parallel/self-loop multigraphs, Lemma 3.1's W(MCB(G)) =
 * W(MCB(G^r)) and dim equality through oracle_reduce).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef struct {
  int32_t n;
  int64_t *start;  /* n+1 */
  int32_t *nbr;    /* 2m (a self-loop appears twice at its vertex) */
  int32_t *eid;    /* edge id of each arc */
} madj_t;

static int madj_build(madj_t *g, int32_t n, int64_t m, const int32_t *src, const int32_t *dst) {
  g->n = n;
  g->start = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  g->nbr = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * m + 1));
  g->eid = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * m + 1));
  if (!g->start || !g->nbr || !g->eid) return -2;
  for (int64_t e = 0; e < m; ++e) { g->start[src[e] + 1]++; g->start[dst[e] + 1]++; }
  for (int32_t v = 0; v < n; ++v) g->start[v + 1] += g->start[v];
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
  if (!fill) return -2;
  memcpy(fill, g->start, sizeof(int64_t) * (size_t)n);
  for (int64_t e = 0; e < m; ++e) {
    g->nbr[fill[src[e]]] = dst[e]; g->eid[fill[src[e]]++] = (int32_t)e;
    g->nbr[fill[dst[e]]] = src[e]; g->eid[fill[dst[e]]++] = (int32_t)e;
  }
  free(fill);
  return 0;
}
static void madj_free(madj_t *g) { free(g->start); free(g->nbr); free(g->eid); }

static int mvalidate(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w) {
  if (n < 1 || m < 0) return -1;
  for (int64_t e = 0; e < m; ++e)
    if (src[e] < 0 || src[e] >= n || dst[e] < 0 || dst[e] >= n || w[e] < 1) return -1;
  return 0;
}

/* ---------------------------------------------------------------- binary heap of (key, vertex) */
typedef struct { int64_t d; int32_t v; } mitem_t;
static void mpush(mitem_t *h, int64_t *sz, mitem_t x) {
  int64_t i = (*sz)++;
  while (i > 0) { int64_t p = (i - 1) / 2; if (h[p].d <= x.d) break; h[i] = h[p]; i = p; }
  h[i] = x;
}
static mitem_t mpop(mitem_t *h, int64_t *sz) {
  mitem_t top = h[0], x = h[--(*sz)];
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

/* Dijkstra from x on the (multi)graph: dist (-1 unreached), parent vertex and parent edge. */
static void mdijkstra(const madj_t *g, const int32_t *w, int32_t x, int64_t *dist, int32_t *par, int32_t *pe,
                      mitem_t *heap) {
  int64_t sz = 0;
  for (int32_t v = 0; v < g->n; ++v) { dist[v] = -1; par[v] = -1; pe[v] = -1; }
  dist[x] = 0;
  mpush(heap, &sz, (mitem_t){0, x});
  while (sz > 0) {
    mitem_t it = mpop(heap, &sz);
    if (it.d != dist[it.v]) continue;
    for (int64_t a = g->start[it.v]; a < g->start[it.v + 1]; ++a) {
      const int32_t u = g->nbr[a];
      const int64_t nd = it.d + w[g->eid[a]];
      if (dist[u] < 0 || nd < dist[u]) {
        dist[u] = nd; par[u] = it.v; pe[u] = g->eid[a];
        mpush(heap, &sz, (mitem_t){nd, u});
      }
    }
  }
}

/* components by union-find */
static int32_t mfind(int32_t *p, int32_t x) { while (p[x] != x) { p[x] = p[p[x]]; x = p[x]; } return x; }
static int32_t mcomponents(int32_t n, int64_t m, const int32_t *src, const int32_t *dst) {
  int32_t *p = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  for (int32_t i = 0; i < n; ++i) p[i] = i;
  int32_t k = n;
  for (int64_t e = 0; e < m; ++e) {
    int32_t a = mfind(p, src[e]), b = mfind(p, dst[e]);
    if (a != b) { p[a] = b; --k; }
  }
  free(p);
  return k;
}

/* ---------------------------------------------------------------- GF(2) basis in echelon form */
typedef struct {
  int64_t words;     /* per vector */
  int32_t rows;
  uint64_t *v;       /* rows x words */
  int64_t *piv;      /* pivot bit of each row */
} gf2_t;

/* reduce x by the basis; returns 1 (and adds it) when x is independent */
static int gf2_insert(gf2_t *B, uint64_t *x) {
  for (int32_t r = 0; r < B->rows; ++r) {
    const int64_t p = B->piv[r];
    if ((x[p >> 6] >> (p & 63)) & 1) {
      const uint64_t *row = B->v + (int64_t)r * B->words;
      for (int64_t k = 0; k < B->words; ++k) x[k] ^= row[k];
    }
  }
  for (int64_t k = 0; k < B->words; ++k)
    if (x[k]) {
      const int64_t p = k * 64 + __builtin_ctzll(x[k]);
      memcpy(B->v + (int64_t)B->rows * B->words, x, sizeof(uint64_t) * (size_t)B->words);
      B->piv[B->rows++] = p;
      return 1;
    }
  return 0;
}

typedef struct { int64_t w; int32_t x; int32_t e; } hcand_t;
static int hcand_cmp(const void *a, const void *b) {
  const hcand_t *p = (const hcand_t *)a, *q = (const hcand_t *)b;
  if (p->w != q->w) return p->w < q->w ? -1 : 1;
  if (p->x != q->x) return p->x < q->x ? -1 : 1;
  return (p->e > q->e) - (p->e < q->e);
}

/* Horton.  Outputs: *weight, *dim (= f); cyc_off[f+1] and cyc_edges[...] (may be NULL) with the edge
 * ids of the kept cycles, cap = capacity of cyc_edges.  Returns 0 or a negative status. */
int oracle_mcb_horton(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w,
                      int64_t *weight, int32_t *dim, int64_t *cyc_off, int32_t *cyc_edges, int64_t cap) {
  if (mvalidate(n, m, src, dst, w)) return -1;
  const int32_t k = mcomponents(n, m, src, dst);
  const int64_t f = m - n + k;
  *dim = (int32_t)f;
  *weight = 0;
  if (cyc_off) cyc_off[0] = 0;
  if (f == 0) return 0;
  madj_t g;
  if (madj_build(&g, n, m, src, dst)) { madj_free(&g); return -2; }
  /* every tree first (n x n int64 distances + parents: small graphs only) */
  int64_t *dist = (int64_t *)malloc(sizeof(int64_t) * (size_t)n * n);
  int32_t *par = (int32_t *)malloc(sizeof(int32_t) * (size_t)n * n);
  int32_t *pe = (int32_t *)malloc(sizeof(int32_t) * (size_t)n * n);
  if (!dist || !par || !pe) return -2;
#pragma omp parallel
  {
    mitem_t *heap = (mitem_t *)malloc(sizeof(mitem_t) * (size_t)(2 * m + 2));
#pragma omp for schedule(dynamic, 8)
    for (int32_t x = 0; x < n; ++x)
      mdijkstra(&g, w, x, dist + (int64_t)x * n, par + (int64_t)x * n, pe + (int64_t)x * n, heap);
    free(heap);
  }
  /* Horton candidates: e = (u, v) not a tree edge of T_x, tree paths from u and v meeting only at x */
  int64_t ncand = 0, capc = 1024;
  hcand_t *cand = (hcand_t *)malloc(sizeof(hcand_t) * (size_t)capc);
  int32_t *mark = (int32_t *)calloc((size_t)n, sizeof(int32_t));
  int32_t stamp = 0;
  for (int32_t x = 0; x < n; ++x) {
    const int64_t *d = dist + (int64_t)x * n;
    const int32_t *px = par + (int64_t)x * n, *ex = pe + (int64_t)x * n;
    for (int64_t e = 0; e < m; ++e) {
      const int32_t u = src[e], v = dst[e];
      if (d[u] < 0) continue;
      int ok;
      if (u == v) {
        ok = (u == x);
      } else if (ex[u] == (int32_t)e || ex[v] == (int32_t)e) {
        ok = 0;
      } else {
        ++stamp;
        for (int32_t a = u; a >= 0; a = px[a]) mark[a] = stamp;
        int32_t a = v;
        while (mark[a] != stamp) a = px[a];
        ok = (a == x);
      }
      if (!ok) continue;
      if (ncand == capc) { capc *= 2; cand = (hcand_t *)realloc(cand, sizeof(hcand_t) * (size_t)capc); }
      cand[ncand++] = (hcand_t){d[u] + w[e] + d[v], x, (int32_t)e};
    }
  }
  qsort(cand, (size_t)ncand, sizeof(hcand_t), hcand_cmp);
  gf2_t B;
  B.words = (m + 63) / 64;
  B.rows = 0;
  B.v = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(B.words * f));
  B.piv = (int64_t *)malloc(sizeof(int64_t) * (size_t)f);
  uint64_t *vec = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)B.words);
  int32_t *cedges = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * n + 2));
  int64_t used = 0;
  int status = 0;
  for (int64_t c = 0; c < ncand && B.rows < f; ++c) {
    const int32_t x = cand[c].x, e = cand[c].e, u = src[e], v = dst[e];
    const int32_t *px = par + (int64_t)x * n, *ex = pe + (int64_t)x * n;
    memset(vec, 0, sizeof(uint64_t) * (size_t)B.words);
    int32_t len = 0;
    cedges[len++] = e;
    if (u != v) {
      for (int32_t a = u; a != x; a = px[a]) cedges[len++] = ex[a];
      for (int32_t a = v; a != x; a = px[a]) cedges[len++] = ex[a];
    }
    for (int32_t i = 0; i < len; ++i) vec[cedges[i] >> 6] ^= 1ull << (cedges[i] & 63);
    if (!gf2_insert(&B, vec)) continue;
    *weight += cand[c].w;
    if (cyc_off) {
      if (cyc_edges) {
        if (used + len > cap) { status = -3; break; }
        memcpy(cyc_edges + used, cedges, sizeof(int32_t) * (size_t)len);
      }
      used += len;
      cyc_off[B.rows] = used;
    }
  }
  if (status == 0 && B.rows != f) status = -4;   /* cannot happen: the Horton set spans the cycle space */
  free(vec); free(cedges); free(B.v); free(B.piv); free(cand); free(mark);
  free(dist); free(par); free(pe);
  madj_free(&g);
  return status;
}

/* de Pina (Algorithm 2) with the signed-graph search of sec. 3.2.1.  Outputs as oracle_mcb_horton,
 * plus wts[f] (weight of C_i in phase order). */
int oracle_mcb_depina(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, const int32_t *w,
                      int64_t *weight, int32_t *dim, int64_t *wts) {
  if (mvalidate(n, m, src, dst, w)) return -1;
  const int32_t k = mcomponents(n, m, src, dst);
  const int64_t f = m - n + k;
  *dim = (int32_t)f;
  *weight = 0;
  if (f == 0) return 0;
  madj_t g;
  if (madj_build(&g, n, m, src, dst)) { madj_free(&g); return -2; }
  /* spanning tree T of the underlying unweighted graph: BFS from the lowest vertex of each component */
  char *intree = (char *)calloc((size_t)m, 1);
  int32_t *seen = (int32_t *)calloc((size_t)n, sizeof(int32_t));
  int32_t *queue = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  for (int32_t r = 0; r < n; ++r) {
    if (seen[r]) continue;
    int32_t qh = 0, qt = 0;
    queue[qt++] = r; seen[r] = 1;
    while (qh < qt) {
      const int32_t a = queue[qh++];
      for (int64_t i = g.start[a]; i < g.start[a + 1]; ++i) {
        const int32_t b = g.nbr[i];
        if (!seen[b]) { seen[b] = 1; intree[g.eid[i]] = 1; queue[qt++] = b; }
      }
    }
  }
  /* E' = non-tree edges in edge order: coordinate of e in the witness space, or -1 */
  int32_t *coord = (int32_t *)malloc(sizeof(int32_t) * (size_t)m);
  int32_t nf = 0;
  for (int64_t e = 0; e < m; ++e) coord[e] = intree[e] ? -1 : nf++;
  const int64_t W = (f + 63) / 64;
  uint64_t *S = (uint64_t *)calloc((size_t)(f * W), sizeof(uint64_t));   /* S_i = e_i (line 1) */
  for (int64_t i = 0; i < f; ++i) S[i * W + (i >> 6)] = 1ull << (i & 63);
  uint64_t *C = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)W);
  int64_t *dist = (int64_t *)malloc(sizeof(int64_t) * (size_t)(2 * n));
  int32_t *pv = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * n));
  int32_t *pa = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * n));
  mitem_t *heap = (mitem_t *)malloc(sizeof(mitem_t) * (size_t)(4 * m + 4));
  int status = 0;
  for (int64_t i = 0; i < f && status == 0; ++i) {   /* line 2 */
    const uint64_t *Si = S + i * W;
    /* line 3: min over x of the shortest x+ -> x- path in the signed graph (sign flips on supp S_i) */
    int64_t best = -1;
    int32_t bx = -1;
    for (int32_t x = 0; x < n; ++x) {
      int64_t sz = 0;
      for (int32_t v = 0; v < 2 * n; ++v) { dist[v] = -1; pv[v] = -1; pa[v] = -1; }
      dist[x] = 0;   /* node v+ is v, v- is n + v */
      mpush(heap, &sz, (mitem_t){0, x});
      while (sz > 0) {
        mitem_t it = mpop(heap, &sz);
        if (it.d != dist[it.v]) continue;
        if (it.v == n + x) break;
        if (best >= 0 && it.d >= best) break;
        const int32_t a = it.v % n, sa = it.v / n;
        for (int64_t q = g.start[a]; q < g.start[a + 1]; ++q) {
          const int32_t e = g.eid[q], b = g.nbr[q];
          const int flip = coord[e] >= 0 && ((Si[coord[e] >> 6] >> (coord[e] & 63)) & 1);
          const int32_t to = (flip ? 1 - sa : sa) * n + b;
          const int64_t nd = it.d + w[e];
          if (dist[to] < 0 || nd < dist[to]) {
            dist[to] = nd; pv[to] = it.v; pa[to] = e;
            mpush(heap, &sz, (mitem_t){nd, to});
          }
        }
      }
      if (dist[n + x] >= 0 && (best < 0 || dist[n + x] < best)) {
        best = dist[n + x];
        bx = x;
        /* the cycle's restriction to E': xor of the walk's non-tree edges */
        memset(C, 0, sizeof(uint64_t) * (size_t)W);
        for (int32_t t = n + x; t != x; t = pv[t]) {
          const int32_t e = pa[t];
          if (coord[e] >= 0) C[coord[e] >> 6] ^= 1ull << (coord[e] & 63);
        }
      }
    }
    if (bx < 0) { status = -4; break; }   /* cannot happen: the fundamental cycle of e_i is odd */
    *weight += best;
    if (wts) wts[i] = best;
    /* lines 4-8: S_j ^= S_i for every later witness not orthogonal to C_i */
    for (int64_t j = i + 1; j < f; ++j) {
      uint64_t *Sj = S + j * W;
      int par = 0;
      for (int64_t q = 0; q < W; ++q) par ^= __builtin_parityll(Sj[q] & C[q]);
      if (par)
        for (int64_t q = 0; q < W; ++q) Sj[q] ^= Si[q];
    }
  }
  free(intree); free(seen); free(queue); free(coord); free(S); free(C); free(dist); free(pv); free(pa); free(heap);
  madj_free(&g);
  return status;
}
