// Expansion-kernel lab (development tool, not product code): candidate designs of Phase III's
// k_expand, timed and compared bit-for-bit against the library's kernel by tools/expand_lab.py.
// It reads the library's plan struct (ear_plan_s from csrc/common.cuh) for the descriptors.
//
//   v1  warp-specialised: 8 producer warps gather R rows (lane-consecutive columns, coalesced
//       gathers) into a 2-deep shared-memory ring, 8 consumer warps stream the output rows with
//       128-bit loads/stores; named barriers (FULL/EMPTY) between the two roles.
//   v9  store ceiling: consumers only, constant output (no gathers) -- the HBM-write bound of this
//       grid/row-group shape.
#include <cstdint>
#include <cstdio>

#include "common.cuh"

namespace lab {
using ear::INF;
using ear::VDesc;

constexpr int RB = 32;   // rows per CTA
constexpr int NC = 256;  // consumer threads (4 columns each)
constexpr int CW = NC * 4;

__device__ __forceinline__ void st_cs_v4(int32_t *p, int4 v) {
  asm volatile("st.global.cs.v4.s32 [%0], {%1, %2, %3, %4};\n" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}
__device__ __forceinline__ void bar_sync(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void bar_arrive(int id, int n) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ int32_t out_val(int32_t cp, int32_t rp, int32_t cq, int32_t rq) {
  return min(__viaddmin_s32(cq, rq, cp + rp), INF);
}

template <int ECAP>
struct Groups {
  VDesc rdesc[RB];
  int32_t ends[2 * RB];
  int8_t ip[RB], iq[RB];
  int8_t sg_row0[RB + 1], sg_e0[RB + 1];
  int32_t n_sg;
};

// greedy partition of the CTA's rows into sub-groups with <= ECAP distinct chain ends (thread 0)
template <int ECAP>
__device__ void make_groups(Groups<ECAP> &G, int nrows) {
  int g = 0, ne = 0, e0 = 0;
  G.sg_row0[0] = 0;
  G.sg_e0[0] = 0;
  for (int r = 0; r < nrows; ++r) {
    const int32_t p = G.rdesc[r].p, q = G.rdesc[r].q;
    int fp = -1, fq = -1;
    for (int e = e0; e < ne; ++e) {
      if (G.ends[e] == p) fp = e;
      if (G.ends[e] == q) fq = e;
    }
    const int need = (fp < 0) + (fq < 0 && q != p);
    if (ne - e0 + need > ECAP) {
      ++g;
      G.sg_row0[g] = (int8_t)r;
      G.sg_e0[g] = (int8_t)ne;
      e0 = ne;
      fp = fq = -1;
    }
    if (fp < 0) { fp = ne; G.ends[ne++] = p; }
    if (fq < 0) {
      if (q == p) fq = fp;
      else { fq = ne; G.ends[ne++] = q; }
    }
    G.ip[r] = (int8_t)(fp - e0);
    G.iq[r] = (int8_t)(fq - e0);
  }
  ++g;
  G.sg_row0[g] = (int8_t)nrows;
  G.sg_e0[g] = (int8_t)ne;
  G.n_sg = g;
}

// v1: warp-specialised producer/consumer
template <int ECAP, int NS, int NP, int MINB>
__global__ void __launch_bounds__(NC + NP * 32, MINB)
    k_ws(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc, int32_t n, int32_t row_begin,
         int32_t row_end, int32_t *__restrict__ out, int64_t ldo) {
  extern __shared__ __align__(16) int32_t R[];   // [NS][ECAP][CW]
  __shared__ Groups<ECAP> G;
  constexpr int NT = NC + NP * 32;
  const int tid = threadIdx.x;
  const int32_t r0 = row_begin + blockIdx.x * RB;
  const int nrows = min(RB, row_end - r0);
  if (tid < nrows) G.rdesc[tid] = desc[r0 + tid];
  __syncthreads();
  if (tid == 0) make_groups<ECAP>(G, nrows);
  __syncthreads();
  const int nsg = G.n_sg;
  const int nchunks = (n + CW - 1) / CW;
  const int total = nchunks * nsg;
  if (tid >= NC) {
    // ---------------- producers: R[e][c] = min(D[e,p_c] + cp_c, D[e,q_c] + cq_c)
    const int pt_ = tid - NC;
    const int lane = pt_ & 31, pw = pt_ >> 5;
    constexpr int CPT = CW / (NP * 32);   // columns per producer thread
    int i = 0;
    for (int c = 0; c < nchunks; ++c) {
      const int32_t c0 = c * CW;
      int32_t pt[CPT], cpt[CPT], qt[CPT], cqt[CPT];
#pragma unroll
      for (int j = 0; j < CPT; ++j) {
        const int32_t t = c0 + (pw * CPT + j) * 32 + lane;
        if (t < n) {
          const VDesc d = desc[t];
          pt[j] = d.p; cpt[j] = d.cp; qt[j] = d.q; cqt[j] = d.cq;
        } else {
          pt[j] = qt[j] = 0; cpt[j] = cqt[j] = 0;
        }
      }
      for (int g = 0; g < nsg; ++g, ++i) {
        const int buf = i % NS;
        if (i >= NS) bar_sync(1 + NS + buf, NT);   // EMPTY[buf]
        int32_t *Rb = R + buf * ECAP * CW;
        const int e0 = G.sg_e0[g], ne = G.sg_e0[g + 1] - e0;
        int e = 0;
        for (; e + 2 <= ne; e += 2) {
          int32_t gp[2][CPT], gq[2][CPT];
#pragma unroll
          for (int u = 0; u < 2; ++u) {
            const int32_t *De = D + (int64_t)G.ends[e0 + e + u] * ldd;
#pragma unroll
            for (int j = 0; j < CPT; ++j) {
              gp[u][j] = __ldg(De + pt[j]);
              gq[u][j] = __ldg(De + qt[j]);
            }
          }
#pragma unroll
          for (int u = 0; u < 2; ++u)
#pragma unroll
            for (int j = 0; j < CPT; ++j)
              Rb[(e + u) * CW + (pw * CPT + j) * 32 + lane] =
                  min(__viaddmin_s32(gq[u][j], cqt[j], gp[u][j] + cpt[j]), INF);
        }
        if (e < ne) {
          const int32_t *De = D + (int64_t)G.ends[e0 + e] * ldd;
#pragma unroll
          for (int j = 0; j < CPT; ++j)
            Rb[e * CW + (pw * CPT + j) * 32 + lane] =
                min(__viaddmin_s32(__ldg(De + qt[j]), cqt[j], __ldg(De + pt[j]) + cpt[j]), INF);
        }
        bar_arrive(1 + buf, NT);   // FULL[buf]
      }
    }
  } else {
    // ---------------- consumers: out rows from R with 128-bit loads and streaming stores
    int i = 0;
    for (int c = 0; c < nchunks; ++c) {
      const int32_t col = c * CW + tid * 4;
      const int ncol = max(0, min(4, n - col));
      const bool vec = (ncol == 4) && ((ldo & 3) == 0);
      for (int g = 0; g < nsg; ++g, ++i) {
        const int buf = i % NS;
        bar_sync(1 + buf, NT);   // FULL[buf]
        const int32_t *Rt = R + buf * ECAP * CW + tid * 4;
        const int rend = G.sg_row0[g + 1];
        int last_p = -1, last_q = -1;
        int4 a = make_int4(0, 0, 0, 0), b = a;
        if (ncol > 0) {
          for (int r = G.sg_row0[g]; r < rend; ++r) {
            const VDesc s = G.rdesc[r];
            const int rp = G.ip[r], rq = G.iq[r];
            if (rp != last_p || rq != last_q) {
              a = *reinterpret_cast<const int4 *>(Rt + rp * CW);
              b = (rq == rp) ? a : *reinterpret_cast<const int4 *>(Rt + rq * CW);
              last_p = rp; last_q = rq;
            }
            int4 o;
            o.x = out_val(s.cp, a.x, s.cq, b.x);
            o.y = out_val(s.cp, a.y, s.cq, b.y);
            o.z = out_val(s.cp, a.z, s.cq, b.z);
            o.w = out_val(s.cp, a.w, s.cq, b.w);
            int32_t *orow = out + (int64_t)(r0 - row_begin + r) * ldo + col;
            if (vec) {
              st_cs_v4(orow, o);
            } else {
              const int32_t ov[4] = {o.x, o.y, o.z, o.w};
              for (int j = 0; j < ncol; ++j) orow[j] = ov[j];
            }
          }
        }
        if (i + NS < total) bar_arrive(1 + NS + buf, NT);   // EMPTY[buf] (only if a producer waits on it)
      }
    }
  }
}

// v9: store ceiling with the same grid (no gathers, no shared memory)
__global__ void __launch_bounds__(NC) k_store_only(int32_t n, int32_t row_begin, int32_t row_end, int32_t *out,
                                                    int64_t ldo) {
  const int32_t r0 = row_begin + blockIdx.x * RB;
  const int nrows = min(RB, row_end - r0);
  for (int32_t c0 = 0; c0 < n; c0 += CW) {
    const int32_t col = c0 + threadIdx.x * 4;
    if (col + 4 > n) break;
    for (int r = 0; r < nrows; ++r)
      st_cs_v4(out + (int64_t)(r0 - row_begin + r) * ldo + col, make_int4(r, col, 1, 2));
  }
}

// v6: warp-local R slices, lane-consecutive (coalesced) gathers, packed row metadata, terminal rows
// of the group emitted straight from the R build (no R reload), chain rows from R with int4 loads.
// meta[r] = {cp, cq, ip | iq << 8, local row}; end_row[e] = local output row of a terminal end that
// lies in the same sub-group, else -1.
template <int ECAP, int MINB>
__global__ void __launch_bounds__(256, MINB)
    k_v6(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc, int32_t n, int32_t row_begin,
         int32_t row_end, int32_t *__restrict__ out, int64_t ldo) {
  extern __shared__ __align__(16) int32_t R[];   // [ECAP][1024]
  __shared__ Groups<ECAP> G;
  __shared__ int4 meta[RB];          // chain rows of each sub-group first-come (terminal rows excluded)
  __shared__ int8_t sg_m0[RB + 1];   // sub-group g: chain rows meta[sg_m0[g] .. sg_m0[g+1])
  __shared__ int16_t end_row[2 * RB];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int32_t r0 = row_begin + blockIdx.x * RB;
  const int nrows = min(RB, row_end - r0);
  if (tid < nrows) G.rdesc[tid] = desc[r0 + tid];
  __syncthreads();
  if (tid == 0) {
    make_groups<ECAP>(G, nrows);
    int m = 0;
    for (int g = 0; g < G.n_sg; ++g) {
      sg_m0[g] = (int8_t)m;
      const int e0 = G.sg_e0[g];
      for (int e = e0; e < G.sg_e0[g + 1]; ++e) end_row[e] = -1;
      for (int r = G.sg_row0[g]; r < G.sg_row0[g + 1]; ++r) {
        const VDesc d = G.rdesc[r];
        if (d.p == d.q && d.cp == 0 && d.cq == 0 && end_row[e0 + G.ip[r]] < 0) {
          end_row[e0 + G.ip[r]] = (int16_t)r;    // terminal row: emitted by the R build
        } else {
          meta[m++] = make_int4(d.cp, d.cq, (int)G.ip[r] | ((int)G.iq[r] << 8), r);
        }
      }
    }
    sg_m0[G.n_sg] = (int8_t)m;
  }
  __syncthreads();
  const int nsg = G.n_sg;
  const bool vec_ok = (ldo & 3) == 0;
  int32_t *Rw = R + w * 128;   // this warp's 128-column slice of every R row
  for (int32_t c0 = w * 128; c0 < n; c0 += 1024) {
    int32_t pt[4], cpt[4], qt[4], cqt[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int32_t t = c0 + 32 * j + lane;
      if (t < n) {
        const VDesc d = desc[t];
        pt[j] = d.p; cpt[j] = d.cp; qt[j] = d.q; cqt[j] = d.cq;
      } else {
        pt[j] = qt[j] = 0; cpt[j] = cqt[j] = 0;
      }
    }
    for (int g = 0; g < nsg; ++g) {
      const int e0 = G.sg_e0[g], ne = G.sg_e0[g + 1] - e0;
      for (int e = 0; e < ne; e += 4) {
        int32_t gp[4][4], gq[4][4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          if (e + u < ne) {
            const int32_t *De = D + (int64_t)G.ends[e0 + e + u] * ldd;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              gp[u][j] = __ldg(De + pt[j]);
              gq[u][j] = __ldg(De + qt[j]);
            }
          }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          if (e + u < ne) {
            const int er = end_row[e0 + e + u];
            int32_t *orow = out + (int64_t)(r0 - row_begin + er) * ldo;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const int32_t v = min(__viaddmin_s32(gq[u][j], cqt[j], gp[u][j] + cpt[j]), INF);
              Rw[(e + u) * 1024 + 32 * j + lane] = v;
              const int32_t t = c0 + 32 * j + lane;
              if (er >= 0 && t < n) __stcs(orow + t, v);
            }
          }
        }
      }
      __syncwarp();
      const int32_t col = c0 + lane * 4;
      const int ncol = max(0, min(4, n - col));
      const int m1 = sg_m0[g + 1];
      int last = -1;
      int4 a = make_int4(0, 0, 0, 0), b = a;
      if (ncol > 0) {
        for (int m = sg_m0[g]; m < m1; ++m) {
          const int4 md = meta[m];
          if (md.z != last) {
            a = *reinterpret_cast<const int4 *>(Rw + (md.z & 0xFF) * 1024 + lane * 4);
            b = *reinterpret_cast<const int4 *>(Rw + (md.z >> 8) * 1024 + lane * 4);
            last = md.z;
          }
          int4 o;
          o.x = out_val(md.x, a.x, md.y, b.x);
          o.y = out_val(md.x, a.y, md.y, b.y);
          o.z = out_val(md.x, a.z, md.y, b.z);
          o.w = out_val(md.x, a.w, md.y, b.w);
          int32_t *orow = out + (int64_t)(r0 - row_begin + md.w) * ldo + col;
          if (ncol == 4 && vec_ok) {
            st_cs_v4(orow, o);
          } else {
            const int32_t ov[4] = {o.x, o.y, o.z, o.w};
            for (int j = 0; j < ncol; ++j) orow[j] = ov[j];
          }
        }
      }
      __syncwarp();
    }
  }
}

// v11: v6 + software pipelining: the gathers of the next end batch (possibly the next sub-group or
// chunk) are in flight while the current batch is turned into R and the sub-group's rows are written.
// Column descriptors of a warp's current/next chunk live in shared memory (cp/cq needed at consume).
struct Item {
  int c, g, b;   // chunk (per warp), sub-group, first end of the batch
};

template <int ECAP, int MINB>
__global__ void __launch_bounds__(256, MINB)
    k_v11(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc, int32_t n, int32_t row_begin,
          int32_t row_end, int32_t *__restrict__ out, int64_t ldo) {
  extern __shared__ __align__(16) int32_t R[];   // [ECAP][1024]
  __shared__ Groups<ECAP> G;
  __shared__ int4 meta[RB];
  __shared__ int8_t sg_m0[RB + 1];
  __shared__ int16_t end_row[2 * RB];
  __shared__ int4 sdesc[8][2][128];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int32_t r0 = row_begin + blockIdx.x * RB;
  const int nrows = min(RB, row_end - r0);
  if (tid < nrows) G.rdesc[tid] = desc[r0 + tid];
  __syncthreads();
  if (tid == 0) {
    make_groups<ECAP>(G, nrows);
    int m = 0;
    for (int g = 0; g < G.n_sg; ++g) {
      sg_m0[g] = (int8_t)m;
      const int e0 = G.sg_e0[g];
      for (int e = e0; e < G.sg_e0[g + 1]; ++e) end_row[e] = -1;
      for (int r = G.sg_row0[g]; r < G.sg_row0[g + 1]; ++r) {
        const VDesc d = G.rdesc[r];
        if (d.p == d.q && d.cp == 0 && d.cq == 0 && end_row[e0 + G.ip[r]] < 0) {
          end_row[e0 + G.ip[r]] = (int16_t)r;
        } else {
          meta[m++] = make_int4(d.cp, d.cq, (int)G.ip[r] | ((int)G.iq[r] << 8), r);
        }
      }
    }
    sg_m0[G.n_sg] = (int8_t)m;
  }
  __syncthreads();
  const int nsg = G.n_sg;
  const bool vec_ok = (ldo & 3) == 0;
  const int nchunk = n > w * 128 ? (n - w * 128 + 1023) / 1024 : 0;
  if (nchunk == 0) return;
  int32_t *Rw = R + w * 128;
  int4 *sd = &sdesc[w][0][0];

  auto next = [&](Item it) {
    it.b += 4;
    if (it.b >= G.sg_e0[it.g + 1] - G.sg_e0[it.g]) {
      it.b = 0;
      if (++it.g == nsg) { it.g = 0; ++it.c; }
    }
    return it;
  };
  int32_t A[4][4][2], B[4][4][2];
  // gathers of item `it` into buffer X
#define V11_ISSUE(X, it)                                                                   \
  do {                                                                                     \
    const int32_t c0_ = w * 128 + (it).c * 1024;                                           \
    int4 *sdc_ = sd + ((it).c & 1) * 128;                                                  \
    int32_t p_[4], q_[4];                                                                  \
    if ((it).g == 0 && (it).b == 0) {                                                      \
      _Pragma("unroll") for (int j = 0; j < 4; ++j) {                                      \
        const int32_t t = c0_ + 32 * j + lane;                                             \
        const VDesc d = t < n ? desc[t] : VDesc{0, 0, 0, 0};                               \
        sdc_[32 * j + lane] = make_int4(d.p, d.cp, d.q, d.cq);                             \
        p_[j] = d.p; q_[j] = d.q;                                                          \
      }                                                                                    \
    } else {                                                                               \
      _Pragma("unroll") for (int j = 0; j < 4; ++j) {                                      \
        const int4 d = sdc_[32 * j + lane];                                                \
        p_[j] = d.x; q_[j] = d.z;                                                          \
      }                                                                                    \
    }                                                                                      \
    const int e0_ = G.sg_e0[(it).g], ne_ = G.sg_e0[(it).g + 1] - e0_;                      \
    _Pragma("unroll") for (int u = 0; u < 4; ++u) {                                        \
      if ((it).b + u < ne_) {                                                              \
        const int32_t *De = D + (int64_t)G.ends[e0_ + (it).b + u] * ldd;                   \
        _Pragma("unroll") for (int j = 0; j < 4; ++j) {                                    \
          X[u][j][0] = __ldg(De + p_[j]);                                                  \
          X[u][j][1] = __ldg(De + q_[j]);                                                  \
        }                                                                                  \
      }                                                                                    \
    }                                                                                      \
  } while (0)

  // R rows of item `it` from buffer X; terminal rows of the group emitted directly; after the last
  // batch of a sub-group, its chain rows are written from R
#define V11_CONSUME(X, it)                                                                 \
  do {                                                                                     \
    const int32_t c0_ = w * 128 + (it).c * 1024;                                           \
    const int4 *sdc_ = sd + ((it).c & 1) * 128;                                            \
    int32_t cp_[4], cq_[4];                                                                \
    _Pragma("unroll") for (int j = 0; j < 4; ++j) {                                        \
      const int4 d = sdc_[32 * j + lane];                                                  \
      cp_[j] = d.y; cq_[j] = d.w;                                                          \
    }                                                                                      \
    const int e0_ = G.sg_e0[(it).g], ne_ = G.sg_e0[(it).g + 1] - e0_;                      \
    _Pragma("unroll") for (int u = 0; u < 4; ++u) {                                        \
      if ((it).b + u < ne_) {                                                              \
        const int er = end_row[e0_ + (it).b + u];                                          \
        int32_t *orow = out + (int64_t)(r0 - row_begin + er) * ldo;                        \
        _Pragma("unroll") for (int j = 0; j < 4; ++j) {                                    \
          const int32_t v = min(__viaddmin_s32(X[u][j][1], cq_[j], X[u][j][0] + cp_[j]), INF); \
          Rw[((it).b + u) * 1024 + 32 * j + lane] = v;                                     \
          const int32_t t = c0_ + 32 * j + lane;                                           \
          if (er >= 0 && t < n) __stcs(orow + t, v);                                       \
        }                                                                                  \
      }                                                                                    \
    }                                                                                      \
    if ((it).b + 4 >= ne_) {                                                               \
      __syncwarp();                                                                        \
      const int32_t col = c0_ + lane * 4;                                                  \
      const int ncol = max(0, min(4, n - col));                                            \
      const int m1 = sg_m0[(it).g + 1];                                                    \
      int last = -1;                                                                       \
      int4 a = make_int4(0, 0, 0, 0), bb = a;                                              \
      if (ncol > 0) {                                                                      \
        for (int m = sg_m0[(it).g]; m < m1; ++m) {                                         \
          const int4 md = meta[m];                                                         \
          if (md.z != last) {                                                              \
            a = *reinterpret_cast<const int4 *>(Rw + (md.z & 0xFF) * 1024 + lane * 4);     \
            bb = *reinterpret_cast<const int4 *>(Rw + (md.z >> 8) * 1024 + lane * 4);      \
            last = md.z;                                                                   \
          }                                                                                \
          int4 o;                                                                          \
          o.x = out_val(md.x, a.x, md.y, bb.x);                                            \
          o.y = out_val(md.x, a.y, md.y, bb.y);                                            \
          o.z = out_val(md.x, a.z, md.y, bb.z);                                            \
          o.w = out_val(md.x, a.w, md.y, bb.w);                                            \
          int32_t *orow = out + (int64_t)(r0 - row_begin + md.w) * ldo + col;              \
          if (ncol == 4 && vec_ok) {                                                       \
            st_cs_v4(orow, o);                                                             \
          } else {                                                                         \
            const int32_t ov[4] = {o.x, o.y, o.z, o.w};                                    \
            for (int j = 0; j < ncol; ++j) orow[j] = ov[j];                                \
          }                                                                                \
        }                                                                                  \
      }                                                                                    \
      __syncwarp();                                                                        \
    }                                                                                      \
  } while (0)

  Item i0{0, 0, 0};
  V11_ISSUE(A, i0);
  while (true) {
    Item i1 = next(i0);
    if (i1.c < nchunk) V11_ISSUE(B, i1);
    __syncwarp();
    V11_CONSUME(A, i0);
    if (i1.c >= nchunk) break;
    i0 = next(i1);
    if (i0.c < nchunk) V11_ISSUE(A, i0);
    __syncwarp();
    V11_CONSUME(B, i1);
    if (i0.c >= nchunk) break;
  }
#undef V11_ISSUE
#undef V11_CONSUME
}

template <int ECAP, int MINB>
int launch_v11(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t rb, int32_t re, int32_t *out, int64_t ldo,
               cudaStream_t st) {
  const int smem = ECAP * 1024 * 4;
  auto k = k_v11<ECAP, MINB>;
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) return -1;
  const int grid = (re - rb + RB - 1) / RB;
  k<<<grid, 256, smem, st>>>(D, ldd, plan->desc, plan->n, rb, re, out, ldo);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// v14: v6 with lean address arithmetic: one 64-bit row pointer per end and 32-bit byte offsets per
// column (2 instructions per gather), a warp-uniform branch for the direct terminal-row emission,
// and output rows addressed by one IMAD.WIDE from a per-lane column base.
__device__ __forceinline__ int32_t ldg_off(const int32_t *base, uint32_t byte_off) {
  return __ldg(reinterpret_cast<const int32_t *>(reinterpret_cast<const char *>(base) + byte_off));
}

__device__ __forceinline__ void prefetch_l2(const void *p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}
__device__ __forceinline__ void prefetch_l2_last(const void *p, uint32_t bytes, uint64_t pol) {
  asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(p), "r"(bytes), "l"(pol) : "memory");
}
// MODE 0: plain; 1: D rows folded onto 64 rows (L2-resident D; wrong values, timing probe);
// 2: sliding bulk L2 prefetch of each end's D-row window two chunks ahead (win[c] = {lo, hi} tids)
template <int ECAP, int MINB, int BATCH, int MODE = 0>
__global__ void __launch_bounds__(256, MINB)
    k_v14(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc, int32_t n, int32_t row_begin,
          int32_t row_end, int32_t *__restrict__ out, int64_t ldo, const int2 *__restrict__ win = nullptr,
          int32_t ldd_pad = 0) {
  extern __shared__ __align__(16) int32_t R[];   // [ECAP][1024]
  __shared__ Groups<ECAP> G;
  __shared__ int4 meta[RB];
  __shared__ int8_t sg_m0[RB + 1];
  __shared__ int16_t end_row[2 * RB];
  __shared__ const int32_t *end_ptr[2 * RB];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int32_t r0 = row_begin + blockIdx.x * RB;
  const int nrows = min(RB, row_end - r0);
  if (tid < nrows) G.rdesc[tid] = desc[r0 + tid];
  __syncthreads();
  if (tid == 0) {
    make_groups<ECAP>(G, nrows);
    int m = 0;
    for (int g = 0; g < G.n_sg; ++g) {
      sg_m0[g] = (int8_t)m;
      const int e0 = G.sg_e0[g];
      for (int e = e0; e < G.sg_e0[g + 1]; ++e) end_row[e] = -1;
      for (int r = G.sg_row0[g]; r < G.sg_row0[g + 1]; ++r) {
        const VDesc d = G.rdesc[r];
        if (d.p == d.q && d.cp == 0 && d.cq == 0 && end_row[e0 + G.ip[r]] < 0) {
          end_row[e0 + G.ip[r]] = (int16_t)r;
        } else {
          meta[m++] = make_int4(d.cp, d.cq, (int)G.ip[r] | ((int)G.iq[r] << 8), r);
        }
      }
    }
    sg_m0[G.n_sg] = (int8_t)m;
  }
  __syncthreads();
  if (tid < G.sg_e0[G.n_sg]) end_ptr[tid] = D + (int64_t)(MODE == 1 ? (G.ends[tid] & 63) : MODE == 3 ? (G.ends[tid] & 255) : MODE == 4 ? (G.ends[tid] & 1023) : MODE == 5 ? (G.ends[tid] & 4095) : G.ends[tid]) * ldd;
  __syncthreads();
  const int nsg = G.n_sg;
  const bool vec_ok = (ldo & 3) == 0;
  const uint32_t ldo_b = (uint32_t)(ldo * 4);
  int32_t *const oblk = out + (int64_t)(r0 - row_begin) * ldo;   // this CTA's first output row
  int32_t *Rw = R + w * 128;
  const int nends = G.sg_e0[nsg];
  const int nchunks = (n + 1023) / 1024;
  constexpr bool PF = MODE == 2 || (MODE >= 6 && MODE <= 8);
  constexpr bool PFT = MODE >= 9;   // per-thread prefetch.global.L2 of the window lines
  constexpr int AHEAD = (MODE == 6 || MODE == 10) ? 1 : MODE == 8 ? 4 : 2;
  constexpr bool LAST = MODE == 7 || MODE == 8;
  uint64_t pol = 0;
  if (LAST) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  if (PF && lane == 0) {   // the first AHEAD chunks up front
    for (int u = w; u < nends; u += 8)
      for (int c = 0; c < AHEAD && c < nchunks; ++c) {
        const int2 wd = win[c];
        if (wd.y > wd.x) {
          if (LAST) prefetch_l2_last(end_ptr[u] + wd.x, (uint32_t)(wd.y - wd.x) * 4u, pol);
          else prefetch_l2(end_ptr[u] + wd.x, (uint32_t)(wd.y - wd.x) * 4u);
        }
      }
  }
  if (PFT) {
    for (int c = 0; c < AHEAD && c < nchunks; ++c) {
      const int2 wd = win[c];
      const int nl = (wd.y - wd.x + 31) >> 5;   // 128-byte lines (approx., window start 16-B aligned)
      for (int u = w; u < nends; u += 8)
        for (int l = lane; l <= nl; l += 32)
          asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(end_ptr[u] + wd.x + 32 * l));
    }
  }
  for (int32_t c0 = w * 128; c0 < n; c0 += 1024) {
    if (PFT) {
      const int cn = (c0 >> 10) + AHEAD;
      if (cn < nchunks) {
        const int2 wd = win[cn];
        const int nl = (wd.y - wd.x + 31) >> 5;
        for (int u = w; u < nends; u += 8)
          for (int l = lane; l <= nl; l += 32)
            asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(end_ptr[u] + wd.x + 32 * l));
      }
    }
    if (PF) {
      const int cn = (c0 >> 10) + AHEAD;
      if (cn < nchunks && lane == 0) {
        const int2 wd = win[cn];
        if (wd.y > wd.x)
          for (int u = w; u < nends; u += 8) {
            if (LAST) prefetch_l2_last(end_ptr[u] + wd.x, (uint32_t)(wd.y - wd.x) * 4u, pol);
            else prefetch_l2(end_ptr[u] + wd.x, (uint32_t)(wd.y - wd.x) * 4u);
          }
      }
    }
    uint32_t op[4], oq[4];
    int32_t cpt[4], cqt[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int32_t t = c0 + 32 * j + lane;
      const VDesc d = t < n ? desc[t] : VDesc{0, 0, 0, 0};
      op[j] = (uint32_t)d.p * 4u; oq[j] = (uint32_t)d.q * 4u; cpt[j] = d.cp; cqt[j] = d.cq;
    }
    for (int g = 0; g < nsg; ++g) {
      const int e0 = G.sg_e0[g], ne = G.sg_e0[g + 1] - e0;
      for (int e = 0; e < ne; e += BATCH) {
        int32_t gp[BATCH][4], gq[BATCH][4];
#pragma unroll
        for (int u = 0; u < BATCH; ++u) {
          const int32_t *De = end_ptr[e0 + min(e + u, ne - 1)];   // past the end: repeat (cached)
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            gp[u][j] = ldg_off(De, op[j]);
            gq[u][j] = ldg_off(De, oq[j]);
          }
        }
#pragma unroll
        for (int u = 0; u < BATCH; ++u) {
          if (e + u < ne) {
            int32_t v[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              v[j] = min(__viaddmin_s32(gq[u][j], cqt[j], gp[u][j] + cpt[j]), INF);
              Rw[(e + u) * 1024 + 32 * j + lane] = v[j];
            }
            const int er = end_row[e0 + e + u];
            if (er >= 0) {   // warp-uniform: a terminal row of this group -- emit it now
              int32_t *orow = reinterpret_cast<int32_t *>(reinterpret_cast<char *>(oblk) + (uint64_t)(uint32_t)er * ldo_b);
#pragma unroll
              for (int j = 0; j < 4; ++j)
                if (c0 + 32 * j + lane < n) __stcs(orow + c0 + 32 * j + lane, v[j]);
            }
          }
        }
      }
      __syncwarp();
      const int32_t col = c0 + lane * 4;
      const int ncol = max(0, min(4, n - col));
      const int m1 = sg_m0[g + 1];
      int32_t *obase = oblk + col;
      int last = -1;
      int4 a = make_int4(0, 0, 0, 0), b = a;
      if (ncol == 4 && vec_ok) {
        for (int m = sg_m0[g]; m < m1; ++m) {
          const int4 md = meta[m];
          if (md.z != last) {
            a = *reinterpret_cast<const int4 *>(Rw + (md.z & 0xFF) * 1024 + lane * 4);
            b = *reinterpret_cast<const int4 *>(Rw + (md.z >> 8) * 1024 + lane * 4);
            last = md.z;
          }
          int4 o;
          o.x = out_val(md.x, a.x, md.y, b.x);
          o.y = out_val(md.x, a.y, md.y, b.y);
          o.z = out_val(md.x, a.z, md.y, b.z);
          o.w = out_val(md.x, a.w, md.y, b.w);
          st_cs_v4(reinterpret_cast<int32_t *>(reinterpret_cast<char *>(obase) + (uint64_t)(uint32_t)md.w * ldo_b), o);
        }
      } else if (ncol > 0) {
        for (int m = sg_m0[g]; m < m1; ++m) {
          const int4 md = meta[m];
          const int32_t *ra = Rw + (md.z & 0xFF) * 1024 + lane * 4, *rb = Rw + (md.z >> 8) * 1024 + lane * 4;
          int32_t *orow = obase + (int64_t)md.w * ldo;
          for (int j = 0; j < ncol; ++j) orow[j] = out_val(md.x, ra[j], md.y, rb[j]);
        }
      }
      __syncwarp();
    }
  }
}

// per 1024-column chunk: the tid range of its terminal columns (contiguous: tids are monotone in
// caller id), widened by 64 and aligned to 16 B
__global__ void k_chunk_windows(const VDesc *__restrict__ desc, int32_t n, int32_t nr, int2 *win) {
  __shared__ int32_t lo, hi;
  const int c = blockIdx.x;
  if (threadIdx.x == 0) { lo = 0x7fffffff; hi = -1; }
  __syncthreads();
  for (int32_t t = c * 1024 + threadIdx.x; t < min(n, c * 1024 + 1024); t += blockDim.x) {
    const VDesc d = desc[t];
    if (d.p == d.q && d.cp == 0) { atomicMin(&lo, d.p); atomicMax(&hi, d.p); }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int2 r = make_int2(0, 0);
    if (hi >= 0) {
      r.x = max(0, lo - 64) & ~3;
      r.y = min(nr, hi + 65);
      r.y = (r.y + 3) & ~3;
    }
    win[c] = r;
  }
}
int2 *g_win = nullptr;

template <int ECAP, int MINB, int BATCH, int MODE = 0>
int launch_v14(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t rb, int32_t re, int32_t *out, int64_t ldo,
               cudaStream_t st) {
  const int smem = ECAP * 1024 * 4;
  auto k = k_v14<ECAP, MINB, BATCH, MODE>;
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) return -1;
  const int grid = (re - rb + RB - 1) / RB;
  if (MODE == 2 || MODE >= 6) {
    const int nch = (plan->n + 1023) / 1024;
    if (!g_win) cudaMalloc(&g_win, sizeof(int2) * (nch + 8));
    k_chunk_windows<<<nch, 256, 0, st>>>(plan->desc, plan->n, plan->n_reduced, g_win);
  }
  k<<<grid, 256, smem, st>>>(D, ldd, plan->desc, plan->n, rb, re, out, ldo, g_win, 0);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// v20: per-128-column-block distinct-tid tables (built once by k_blk_tables): a warp gathers only the
// distinct D[e, x] of its block (sorted tids -> few sectors, no duplicate requests), stages them in
// a per-warp shared table, then expands R rows from it by 8-bit indices.
constexpr int UB = 256;   // max distinct tids per 128-column block (2 per column)

__global__ void __launch_bounds__(256) k_blk_tables(const VDesc *__restrict__ desc, int32_t n, int32_t *U, int32_t *ucnt,
                                                    uint16_t *idx) {
  __shared__ int32_t v[256];
  __shared__ int32_t rnk[256];
  __shared__ int32_t cnt;
  const int b = blockIdx.x, tid = threadIdx.x;
  const int32_t t = b * 128 + (tid & 127);
  int32_t x = 0x7fffffff;
  if (t < n) x = (tid < 128) ? desc[t].p : desc[t].q;
  v[tid] = x;
  if (tid == 0) cnt = 0;
  __syncthreads();
  // first occurrence flags, then rank = number of distinct values below x
  __shared__ int8_t fst[256];
  bool first = true;
  for (int i = 0; i < tid; ++i)
    if (v[i] == x) { first = false; break; }
  fst[tid] = first;
  __syncthreads();
  int r = 0;
  for (int i = 0; i < 256; ++i) r += (fst[i] && v[i] < x);
  rnk[tid] = r;
  if (first && x != 0x7fffffff) {
    U[(int64_t)b * UB + r] = x;
    atomicMax(&cnt, r + 1);
  }
  __syncthreads();
  const int c = cnt;
  // pad the table with its last value (valid addresses for the padded gathers)
  if (tid >= c && c > 0) U[(int64_t)b * UB + tid] = U[(int64_t)b * UB + c - 1];
  if (tid == 0) ucnt[b] = c;
  if (tid < 128 && t < n) idx[t] = (uint16_t)(rnk[tid] | (rnk[tid + 128] << 8));
}

template <int ECAP, int MINB>
__global__ void __launch_bounds__(256, MINB)
    k_v20(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc, const int32_t *__restrict__ U,
          const int32_t *__restrict__ ucnt, const uint16_t *__restrict__ idx, int32_t n, int32_t row_begin,
          int32_t row_end, int32_t *__restrict__ out, int64_t ldo) {
  extern __shared__ __align__(16) int32_t R[];   // [ECAP][1024] then per-warp G tables [8][4][UB]
  __shared__ Groups<ECAP> G;
  __shared__ int4 meta[RB];
  __shared__ int8_t sg_m0[RB + 1];
  __shared__ int16_t end_row[2 * RB];
  __shared__ const int32_t *end_ptr[2 * RB];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int32_t r0 = row_begin + blockIdx.x * RB;
  const int nrows = min(RB, row_end - r0);
  if (tid < nrows) G.rdesc[tid] = desc[r0 + tid];
  __syncthreads();
  if (tid == 0) {
    make_groups<ECAP>(G, nrows);
    int m = 0;
    for (int g = 0; g < G.n_sg; ++g) {
      sg_m0[g] = (int8_t)m;
      const int e0 = G.sg_e0[g];
      for (int e = e0; e < G.sg_e0[g + 1]; ++e) end_row[e] = -1;
      for (int r = G.sg_row0[g]; r < G.sg_row0[g + 1]; ++r) {
        const VDesc d = G.rdesc[r];
        if (d.p == d.q && d.cp == 0 && d.cq == 0 && end_row[e0 + G.ip[r]] < 0) {
          end_row[e0 + G.ip[r]] = (int16_t)r;
        } else {
          meta[m++] = make_int4(d.cp, d.cq, (int)G.ip[r] | ((int)G.iq[r] << 8), r);
        }
      }
    }
    sg_m0[G.n_sg] = (int8_t)m;
  }
  __syncthreads();
  if (tid < G.sg_e0[G.n_sg]) end_ptr[tid] = D + (int64_t)G.ends[tid] * ldd;
  __syncthreads();
  const int nsg = G.n_sg;
  const bool vec_ok = (ldo & 3) == 0;
  const uint32_t ldo_b = (uint32_t)(ldo * 4);
  int32_t *const oblk = out + (int64_t)(r0 - row_begin) * ldo;
  int32_t *Rw = R + w * 128;
  int32_t *Gw = R + ECAP * 1024 + w * 4 * UB;   // this warp's G table for a batch of 4 ends
  for (int32_t c0 = w * 128; c0 < n; c0 += 1024) {
    const int blk = c0 >> 7;
    const int nk = (ucnt[blk] + 31) >> 5;   // warp-uniform
    uint32_t uo[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) uo[k] = k < nk ? (uint32_t)U[(int64_t)blk * UB + k * 32 + lane] * 4u : 0u;
    int32_t cpt[4], cqt[4], ipt[4], iqt[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int32_t t = c0 + 32 * j + lane;
      const VDesc d = t < n ? desc[t] : VDesc{0, 0, 0, 0};
      const uint32_t ix = t < n ? idx[t] : 0u;
      cpt[j] = d.cp; cqt[j] = d.cq; ipt[j] = ix & 0xFF; iqt[j] = ix >> 8;
    }
    for (int g = 0; g < nsg; ++g) {
      const int e0 = G.sg_e0[g], ne = G.sg_e0[g + 1] - e0;
      for (int e = 0; e < ne; e += 4) {
        int32_t gv[4][8];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int32_t *De = end_ptr[e0 + min(e + u, ne - 1)];
#pragma unroll
          for (int k = 0; k < 8; ++k)
            if (k < nk) gv[u][k] = ldg_off(De, uo[k]);
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
          for (int k = 0; k < 8; ++k)
            if (k < nk) Gw[u * UB + k * 32 + lane] = gv[u][k];
        __syncwarp();
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          if (e + u < ne) {
            int32_t v[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              v[j] = min(__viaddmin_s32(Gw[u * UB + iqt[j]], cqt[j], Gw[u * UB + ipt[j]] + cpt[j]), INF);
              Rw[(e + u) * 1024 + 32 * j + lane] = v[j];
            }
            const int er = end_row[e0 + e + u];
            if (er >= 0) {
              int32_t *orow = reinterpret_cast<int32_t *>(reinterpret_cast<char *>(oblk) + (uint64_t)(uint32_t)er * ldo_b);
#pragma unroll
              for (int j = 0; j < 4; ++j)
                if (c0 + 32 * j + lane < n) __stcs(orow + c0 + 32 * j + lane, v[j]);
            }
          }
        }
        __syncwarp();
      }
      const int32_t col = c0 + lane * 4;
      const int ncol = max(0, min(4, n - col));
      const int m1 = sg_m0[g + 1];
      int32_t *obase = oblk + col;
      int last = -1;
      int4 a = make_int4(0, 0, 0, 0), b = a;
      if (ncol == 4 && vec_ok) {
        for (int m = sg_m0[g]; m < m1; ++m) {
          const int4 md = meta[m];
          if (md.z != last) {
            a = *reinterpret_cast<const int4 *>(Rw + (md.z & 0xFF) * 1024 + lane * 4);
            b = *reinterpret_cast<const int4 *>(Rw + (md.z >> 8) * 1024 + lane * 4);
            last = md.z;
          }
          int4 o;
          o.x = out_val(md.x, a.x, md.y, b.x);
          o.y = out_val(md.x, a.y, md.y, b.y);
          o.z = out_val(md.x, a.z, md.y, b.z);
          o.w = out_val(md.x, a.w, md.y, b.w);
          st_cs_v4(reinterpret_cast<int32_t *>(reinterpret_cast<char *>(obase) + (uint64_t)(uint32_t)md.w * ldo_b), o);
        }
      } else if (ncol > 0) {
        for (int m = sg_m0[g]; m < m1; ++m) {
          const int4 md = meta[m];
          const int32_t *ra = Rw + (md.z & 0xFF) * 1024 + lane * 4, *rb = Rw + (md.z >> 8) * 1024 + lane * 4;
          int32_t *orow = obase + (int64_t)md.w * ldo;
          for (int j = 0; j < ncol; ++j) orow[j] = out_val(md.x, ra[j], md.y, rb[j]);
        }
      }
      __syncwarp();
    }
  }
}

struct V20Tables {
  int32_t *U = nullptr, *cnt = nullptr;
  uint16_t *idx = nullptr;
  const void *plan = nullptr;
};
V20Tables g_v20;

template <int ECAP, int MINB>
int launch_v20(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t rb, int32_t re, int32_t *out, int64_t ldo,
               cudaStream_t st) {
  const int32_t n = plan->n;
  const int nblk = (n + 127) / 128;
  if (g_v20.plan != plan) {
    if (g_v20.U) { cudaFree(g_v20.U); cudaFree(g_v20.cnt); cudaFree(g_v20.idx); }
    cudaMalloc(&g_v20.U, (size_t)nblk * UB * 4);
    cudaMalloc(&g_v20.cnt, (size_t)nblk * 4);
    cudaMalloc(&g_v20.idx, (size_t)n * 2);
    g_v20.plan = plan;
  }
  k_blk_tables<<<nblk, 256, 0, st>>>(plan->desc, n, g_v20.U, g_v20.cnt, g_v20.idx);
  const int smem = ECAP * 1024 * 4 + 8 * 4 * UB * 4;
  auto k = k_v20<ECAP, MINB>;
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) return -1;
  const int grid = (re - rb + RB - 1) / RB;
  k<<<grid, 256, smem, st>>>(D, ldd, plan->desc, g_v20.U, g_v20.cnt, g_v20.idx, n, rb, re, out, ldo);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

__global__ void k_same_chain(const VDesc *__restrict__ desc, const int32_t *__restrict__ seg_of,
                             const int32_t *__restrict__ seg_start, const int32_t *__restrict__ seg_vert,
                             int32_t row_begin, int32_t row_end, int32_t *out, int64_t ldo) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t s = row_begin + warp; s < row_end; s += nwarps) {
    const int32_t g = seg_of[s];
    if (g < 0) continue;
    const int32_t off_s = desc[s].cp;
    int32_t *orow = out + (s - row_begin) * ldo;
    for (int32_t i = seg_start[g] + lane; i < seg_start[g + 1]; i += 32) {
      const int32_t t = seg_vert[i];
      const int32_t along = abs(off_s - desc[t].cp);
      if (along < orow[t]) orow[t] = along;
    }
  }
}

void same_chain(const ear_plan_s *plan, int32_t rb, int32_t re, int32_t *out, int64_t ldo, cudaStream_t st) {
  if (plan->n_chain_vertices > 0)
    k_same_chain<<<148 * 16, 256, 0, st>>>(plan->desc, plan->seg_of, plan->seg_start, plan->seg_vert, rb, re, out, ldo);
}

template <int ECAP, int MINB>
int launch_v6(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t rb, int32_t re, int32_t *out, int64_t ldo,
              cudaStream_t st) {
  const int smem = ECAP * 1024 * 4;
  auto k = k_v6<ECAP, MINB>;
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) return -1;
  const int grid = (re - rb + RB - 1) / RB;
  k<<<grid, 256, smem, st>>>(D, ldd, plan->desc, plan->n, rb, re, out, ldo);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

template <int ECAP, int NS, int NP, int MINB>
int launch_ws(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t rb, int32_t re, int32_t *out, int64_t ldo,
              cudaStream_t st) {
  constexpr int NT = NC + NP * 32;
  const int smem = NS * ECAP * CW * 4;
  auto k = k_ws<ECAP, NS, NP, MINB>;
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) return -1;
  const int grid = (re - rb + RB - 1) / RB;
  k<<<grid, NT, smem, st>>>(D, ldd, plan->desc, plan->n, rb, re, out, ldo);
  same_chain(plan, rb, re, out, ldo, st);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

}  // namespace lab

extern "C" int lab_expand(int variant, const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t rb, int32_t re,
                          int32_t *out, int64_t ldo, void *stream) {
  cudaStream_t st = (cudaStream_t)stream;
  using namespace lab;
  switch (variant) {
    case 1: return launch_ws<8, 2, 8, 2>(plan, D, ldd, rb, re, out, ldo, st);
    case 2: return launch_ws<16, 2, 8, 1>(plan, D, ldd, rb, re, out, ldo, st);
    case 3: return launch_ws<8, 2, 4, 2>(plan, D, ldd, rb, re, out, ldo, st);
    case 4: return launch_ws<8, 3, 8, 1>(plan, D, ldd, rb, re, out, ldo, st);
    case 5: return launch_ws<4, 4, 8, 2>(plan, D, ldd, rb, re, out, ldo, st);
    case 6: { int r = launch_v6<16, 3>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 7: { int r = launch_v6<8, 4>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 8: { int r = launch_v6<24, 2>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 10: { int r = launch_v6<16, 2>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 11: { int r = launch_v11<16, 2>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 12: { int r = launch_v11<8, 2>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 13: { int r = launch_v11<24, 2>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 14: { int r = launch_v14<16, 2, 4>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 15: { int r = launch_v14<16, 3, 4>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 16: { int r = launch_v14<16, 2, 8>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 17: { int r = launch_v14<8, 4, 4>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 18: { int r = launch_v14<24, 2, 4>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 20: { int r = launch_v20<16, 2>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 21: { int r = launch_v20<8, 3>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 22: { int r = launch_v20<12, 2>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 23: { int r = launch_v14<16, 2, 4, 1>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 24: { int r = launch_v14<16, 2, 4, 2>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 25: { int r = launch_v14<16, 2, 4, 3>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 26: { int r = launch_v14<16, 2, 4, 4>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 27: { int r = launch_v14<16, 2, 4, 5>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 28: { int r = launch_v14<16, 2, 4, 6>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 29: { int r = launch_v14<16, 2, 4, 7>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 30: { int r = launch_v14<16, 2, 4, 8>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 31: { int r = launch_v14<16, 2, 4, 9>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 32: { int r = launch_v14<16, 2, 4, 10>(plan, D, ldd, rb, re, out, ldo, st); same_chain(plan, rb, re, out, ldo, st); return r; }
    case 9: {
      const int grid = (re - rb + RB - 1) / RB;
      k_store_only<<<grid, NC, 0, st>>>(plan->n, rb, re, out, ldo);
      return cudaGetLastError() == cudaSuccess ? 0 : -2;
    }
  }
  return -3;
}
