// Phase III -- UPDATE_DISTANCE for every row (Alg. 1 lines 9-11; rules P:105-117).
//
// For output row s (caller order) and column t, with per-vertex descriptors
// (p, cp, q, cq) = (tid(left), along-chain distance to it, tid(right), distance to it)
// (terminals: p = q = own tid, cp = cq = 0):
//     R[e, t]   = min(D[e, p_t] + cp_t, D[e, q_t] + cq_t)            2-term rule seen from t
//     S[s, t]   = min(cp_s + R[p_s, t], cq_s + R[q_s, t])            4-term rule; for a
//                                                                    terminal s it is R[tid(s), t]
//                                                                    and for terminal s,t D
//     same chain: S[s, t] = min(S[s, t], |off_s - off_t|)            P:107 (readings C8, C9)
// then clamped to EAR_INF.
//
// k_expand: one CTA per group of RB = 32 consecutive output rows.  The group's distinct chain
// ends E (<= 64) are split greedily into sub-groups of <= ECAP endpoints; for every 1024-column
// chunk each thread owns 4 consecutive columns: it builds R[e, its 4 columns] for the sub-group's
// endpoints in shared memory (2 gathers from the D rows of e each -- the D rows of neighbouring
// rows' endpoints stay in L1/L2 because caller ids are spatially coherent), then emits every row of
// the sub-group with two 128-bit shared loads, 3 integer ops per element and one 128-bit streaming
// store (st.global.cs).  The output is written exactly once: the kernel is HBM-write bound.
// k_same_chain: the P:107 along-chain patch, one warp per row, touching only same-chain entries.
#include <algorithm>

#include "common.cuh"

namespace ear {
namespace {

constexpr int NT = 256;
constexpr int RB = 32;              // rows per CTA
constexpr int ECAP = 16;            // endpoints per sub-group (R tile: ECAP x 1024 ints = 64 KB)
constexpr int CHUNK = NT * 4;       // columns per chunk
constexpr int EXP_SMEM = ECAP * CHUNK * 4;

__device__ __forceinline__ void st_cs_v4(int32_t *p, int4 v) {
  asm volatile("st.global.cs.v4.s32 [%0], {%1, %2, %3, %4};\n" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}

__device__ __forceinline__ int32_t out_val(int32_t cp, int32_t rp, int32_t cq, int32_t rq) {
  // min(cp + rp, cq + rq, INF); every term < 2^31 (cp, cq < 2^30 by the EAR_EOVERFLOW check)
  return min(__viaddmin_s32(cq, rq, cp + rp), INF);
}

template <bool VEC>
__global__ void __launch_bounds__(NT, 3) k_expand(const int32_t *__restrict__ D, int64_t ldd,
                                                 const VDesc *__restrict__ desc, int32_t n, int32_t row_begin,
                                                 int32_t row_end, int32_t *__restrict__ out, int64_t ldo) {
  extern __shared__ __align__(16) int32_t R[];       // [ECAP][CHUNK]
  __shared__ VDesc rdesc[RB];
  __shared__ int32_t ends[2 * RB];                   // endpoint tids, sub-group by sub-group
  __shared__ int8_t ip[RB], iq[RB];                  // per row: index of p / q in its sub-group
  __shared__ int8_t sg_row0[RB + 1], sg_e0[RB + 1];  // sub-group g: rows [row0[g], row0[g+1]), ends [e0[g], e0[g+1])
  __shared__ int32_t n_sg;

  const int tid = threadIdx.x;
  const int32_t r0 = row_begin + blockIdx.x * RB;
  const int nrows = min(RB, row_end - r0);
  if (tid < nrows) rdesc[tid] = desc[r0 + tid];
  __syncthreads();
  if (tid == 0) {
    // greedy partition of the rows into sub-groups with <= ECAP distinct endpoints
    int g = 0, ne = 0, e0 = 0;
    sg_row0[0] = 0; sg_e0[0] = 0;
    for (int r = 0; r < nrows; ++r) {
      const int32_t p = rdesc[r].p, q = rdesc[r].q;
      int fp = -1, fq = -1;
      for (int e = e0; e < ne; ++e) {
        if (ends[e] == p) fp = e;
        if (ends[e] == q) fq = e;
      }
      const int need = (fp < 0) + (fq < 0 && q != p);
      if (ne - e0 + need > ECAP) {   // close the current sub-group
        ++g;
        sg_row0[g] = (int8_t)r; sg_e0[g] = (int8_t)ne; e0 = ne;
        fp = fq = -1;
      }
      if (fp < 0) { fp = ne; ends[ne++] = p; }
      if (fq < 0) {
        if (q == p) fq = fp; else { fq = ne; ends[ne++] = q; }
      }
      ip[r] = (int8_t)(fp - e0); iq[r] = (int8_t)(fq - e0);
    }
    ++g;
    sg_row0[g] = (int8_t)nrows; sg_e0[g] = (int8_t)ne;
    n_sg = g;
  }
  __syncthreads();
  const int nsg = n_sg;
  int32_t *Rt = R + tid * 4;   // this thread's 4 columns in every R row

  for (int32_t c0 = 0; c0 < n; c0 += CHUNK) {
    const int32_t col = c0 + tid * 4;
    if (col >= n) break;   // (no barriers below: every thread works on its own columns only)
    const int ncol = min(4, n - col);
    int32_t pt[4], cpt[4], qt[4], cqt[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (j < ncol) {
        const VDesc d = desc[col + j];
        pt[j] = d.p; cpt[j] = d.cp; qt[j] = d.q; cqt[j] = d.cq;
      } else {
        pt[j] = qt[j] = 0; cpt[j] = cqt[j] = 0;
      }
    }
    for (int g = 0; g < nsg; ++g) {
      const int e0 = sg_e0[g], ne = sg_e0[g + 1] - e0;
      // R rows for the sub-group's endpoints; 4 endpoints per batch keep 32 independent gathers
      // in flight per thread (the kernel is otherwise gather-latency bound)
      int e = 0;
      for (; e + 4 <= ne; e += 4) {
        int32_t gp[4][4], gq[4][4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int32_t *De = D + (int64_t)ends[e0 + e + u] * ldd;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            gp[u][j] = __ldg(De + pt[j]);
            gq[u][j] = __ldg(De + qt[j]);
          }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          int4 v;   // clamped to INF so that cp_s + R below cannot overflow
          v.x = min(__viaddmin_s32(gq[u][0], cqt[0], gp[u][0] + cpt[0]), INF);
          v.y = min(__viaddmin_s32(gq[u][1], cqt[1], gp[u][1] + cpt[1]), INF);
          v.z = min(__viaddmin_s32(gq[u][2], cqt[2], gp[u][2] + cpt[2]), INF);
          v.w = min(__viaddmin_s32(gq[u][3], cqt[3], gp[u][3] + cpt[3]), INF);
          *reinterpret_cast<int4 *>(Rt + (e + u) * CHUNK) = v;
        }
      }
      for (; e < ne; ++e) {
        const int32_t *De = D + (int64_t)ends[e0 + e] * ldd;
        int4 v;
        v.x = min(__viaddmin_s32(__ldg(De + qt[0]), cqt[0], __ldg(De + pt[0]) + cpt[0]), INF);
        v.y = min(__viaddmin_s32(__ldg(De + qt[1]), cqt[1], __ldg(De + pt[1]) + cpt[1]), INF);
        v.z = min(__viaddmin_s32(__ldg(De + qt[2]), cqt[2], __ldg(De + pt[2]) + cpt[2]), INF);
        v.w = min(__viaddmin_s32(__ldg(De + qt[3]), cqt[3], __ldg(De + pt[3]) + cpt[3]), INF);
        *reinterpret_cast<int4 *>(Rt + e * CHUNK) = v;
      }
      const int rend = sg_row0[g + 1];
      int last_p = -1, last_q = -1;
      int4 a = make_int4(0, 0, 0, 0), b = a;
      for (int r = sg_row0[g]; r < rend; ++r) {
        const VDesc s = rdesc[r];
        const int rp = ip[r], rq = iq[r];
        if (rp != last_p || rq != last_q) {   // consecutive rows of one chain share their R rows
          a = *reinterpret_cast<const int4 *>(Rt + rp * CHUNK);
          b = (rq == rp) ? a : *reinterpret_cast<const int4 *>(Rt + rq * CHUNK);   // terminal rows: one load
          last_p = rp; last_q = rq;
        }
        int4 o;
        o.x = out_val(s.cp, a.x, s.cq, b.x);
        o.y = out_val(s.cp, a.y, s.cq, b.y);
        o.z = out_val(s.cp, a.z, s.cq, b.z);
        o.w = out_val(s.cp, a.w, s.cq, b.w);
        int32_t *orow = out + (int64_t)(r0 - row_begin + r) * ldo + col;
        if (VEC && ncol == 4) {
          st_cs_v4(orow, o);
        } else {
          const int32_t ov[4] = {o.x, o.y, o.z, o.w};
#pragma unroll
          for (int j = 0; j < 4; ++j)
            if (j < ncol) orow[j] = ov[j];
        }
      }
    }
  }
}

// P:107 along-chain rule for same-chain pairs (C8: same chain id; C9: min with |off_s - off_t|)
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

// Compact / query mode: S[s,t] for arbitrary pairs from D and the descriptors
// alone -- UPDATE_DISTANCE evaluated per pair, O(N_r^2 + N) memory instead of N^2.
__global__ void k_query_pairs(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc,
                              const int32_t *__restrict__ ear, int64_t npairs, const int32_t *__restrict__ qs,
                              const int32_t *__restrict__ qt, int32_t *__restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < npairs; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t s = qs[i], t = qt[i];
    const VDesc a = desc[s], b = desc[t];
    const int32_t *Dp = D + (int64_t)a.p * ldd, *Dq = D + (int64_t)a.q * ldd;
    // R[e,t] for e in {p_s, q_s} (2-term), then the 4-term rule
    const int32_t rp = min(__viaddmin_s32(Dp[b.q], b.cq, Dp[b.p] + b.cp), INF);
    const int32_t rq = min(__viaddmin_s32(Dq[b.q], b.cq, Dq[b.p] + b.cp), INF);
    int32_t v = min(__viaddmin_s32(a.cq, rq, a.cp + rp), INF);
    const int32_t es = ear[s];
    if (es >= 0 && es == ear[t]) v = min(v, abs(a.cp - b.cp));   // same chain (C8/C9)
    out[i] = v;
  }
}


bool g_attr_set = false;

}  // namespace

ear_status_t expand(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t row_begin, int32_t row_end,
                    int32_t *out, int64_t ldo, cudaStream_t st) {
  const int32_t rows = row_end - row_begin;
  if (rows <= 0) return EAR_OK;
  if (!g_attr_set) {
    EAR_CUDA_TRY(cudaFuncSetAttribute(k_expand<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, EXP_SMEM));
    EAR_CUDA_TRY(cudaFuncSetAttribute(k_expand<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, EXP_SMEM));
    g_attr_set = true;
  }
  const bool vec = ((uintptr_t)out % 16 == 0) && (ldo % 4 == 0);
  const unsigned grid = (unsigned)ceil_div(rows, RB);
  const double nr = plan->n_reduced;
  int se = prof_begin(PK_EXPAND, st);
  if (vec)
    EAR_LAUNCH(k_expand<true>, grid, NT, EXP_SMEM, st)(D, ldd, plan->desc, plan->n, row_begin, row_end, out, ldo);
  else
    EAR_LAUNCH(k_expand<false>, grid, NT, EXP_SMEM, st)(D, ldd, plan->desc, plan->n, row_begin, row_end, out, ldo);
  prof_end(se, st, 4.0 * rows * plan->n + 16.0 * plan->n + 4.0 * nr * nr * rows / plan->n);
  if (plan->n_chain_vertices > 0) {
    int ss = prof_begin(PK_SAME_CHAIN, st);
    const int g2 = (int)std::min<int64_t>(ceil_div((int64_t)rows * 32, 256), 148 * 16);
    EAR_LAUNCH(k_same_chain, g2, 256, 0, st)(plan->desc, plan->seg_of, plan->seg_start, plan->seg_vert, row_begin,
                                      row_end, out, ldo);
    prof_end(ss, st, 0);
  }
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

ear_status_t query_pairs(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int64_t npairs, const int32_t *qs,
                         const int32_t *qt, int32_t *out, cudaStream_t st) {
  if (npairs <= 0) return EAR_OK;
  const int grid = (int)std::min<int64_t>(ceil_div(npairs, 256), 148 * 16);
  EAR_LAUNCH(k_query_pairs, grid, 256, 0, st)(D, ldd, plan->desc, plan->ear, npairs, qs, qt, out);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

}  // namespace ear
