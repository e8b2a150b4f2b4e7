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
// k_expand: persistent CTAs take work items in order -- a group of RB = 32 consecutive output rows
// (the last ~wave of groups split into column segments); a group's distinct chain ends E (<= 64)
// are split greedily into sub-groups of <= ECAP endpoints.  Each of the 8 warps owns a 128-column
// slice of every 1,024-column chunk and works independently of the others (no CTA barrier in the
// main loop):
//   R build   for each end e of the sub-group (4 ends per batch, 32 gathers in flight per lane) and
//             the slice's columns t -- lane-consecutive, so one gather instruction covers 32
//             neighbouring columns and few sectors -- R[e, t] = min(D[e,p_t] + cp_t, D[e,q_t] + cq_t)
//             (2-term rule seen from t) goes to shared memory.  Gathers use one 64-bit row
//             pointer per end and 32-bit byte offsets per column (2 address instructions each).
//             When e is itself a terminal row of the sub-group, R[e, .] IS that output row:
//             it is streamed out right here, never reloaded.
//   rows      every chain row s of the sub-group: S[s, t] = min(cp_s + R[p_s,t], cq_s + R[q_s,t])
//             (4-term rule) with two 128-bit shared loads (shared by consecutive rows of one
//             chain), three integer ops per element and one 128-bit streaming store; row metadata
//             is one packed int4 per row.
// The output is written exactly once.  Measured on cfg4 (tools/expand_lab.py, profiles/): the D
// gathers go to HBM at the first touch of each sector and their latency is what bounds the kernel;
// with D resident in L2 the same kernel runs at ~90 % of the copy bandwidth.
// k_same_chain: the P:107 along-chain patch, one warp per row, touching only same-chain entries.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdlib>

#include "common.cuh"

namespace ear {
namespace {

constexpr int NT = 256;
constexpr int RB = 32;              // rows per CTA
constexpr int ECAP = 16;            // endpoints per sub-group (R tile: ECAP x 1024 ints = 64 KB)
constexpr int CHUNK = 1024;         // columns per chunk (8 warps x 128)
constexpr int BATCH = 4;            // ends per gather batch
#ifndef EXP_MINB
#define EXP_MINB 2
#endif
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

__device__ __forceinline__ int32_t ldg_off(const int32_t *base, uint32_t byte_off) {
  return __ldg(reinterpret_cast<const int32_t *>(reinterpret_cast<const char *>(base) + byte_off));
}

__device__ __forceinline__ int32_t *row_ptr(int32_t *base, int32_t r, uint32_t ld_bytes) {
  return reinterpret_cast<int32_t *>(reinterpret_cast<char *>(base) + (uint64_t)(uint32_t)r * ld_bytes);
}

// Work items, taken in order from a global counter by persistent CTAs (one wave): items [0, n_full)
// are whole row groups (all n columns); the last row groups -- about one wave of them -- are split
// into nseg column segments of seg_w columns (a multiple of CHUNK), so the launch ends with small
// items instead of a partial wave of whole row groups.
struct ExpandWork {
  int32_t *counter;
  int32_t n_full, n_items, nseg, seg_w;
};

__global__ void __launch_bounds__(NT, EXP_MINB) k_expand(const int32_t *__restrict__ D, int64_t ldd,
                                                 const VDesc *__restrict__ desc, int32_t n, int32_t row_begin,
                                                 int32_t row_end, int32_t *__restrict__ out, int64_t ldo,
                                                 const ExpandWork W) {
  extern __shared__ __align__(16) int32_t R[];       // [ECAP][CHUNK]
  __shared__ VDesc rdesc[RB];
  __shared__ int32_t ends[2 * RB];                   // endpoint tids, sub-group by sub-group
  __shared__ const int32_t *end_ptr[2 * RB];         // their D rows
  __shared__ int16_t end_row[2 * RB];                // local output row of a terminal end in its sub-group, or -1
  __shared__ int8_t ip[RB], iq[RB];                  // per row: index of p / q in its sub-group
  __shared__ int8_t sg_row0[RB + 1], sg_e0[RB + 1];  // sub-group g: rows [row0[g], row0[g+1]), ends [e0[g], e0[g+1])
  __shared__ int4 meta[RB];                          // chain rows by sub-group: {cp, cq, ip | iq << 8, local row}
  __shared__ int8_t sg_m0[RB + 1];
  __shared__ int32_t n_sg, item_sh;

  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  for (;;) {
  if (tid == 0) item_sh = atomicAdd(W.counter, 1);
  __syncthreads();
  const int32_t item = item_sh;
  if (item >= W.n_items) break;
  int32_t rg = item, col_b = 0, col_e = n;
  if (item >= W.n_full) {
    rg = W.n_full + (item - W.n_full) / W.nseg;
    col_b = ((item - W.n_full) % W.nseg) * W.seg_w;
    col_e = min(n, col_b + W.seg_w);
  }
  const int32_t r0 = row_begin + rg * RB;
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
    // terminal rows are emitted by the R build of their own end; the rest become chain-row metadata
    int m = 0;
    for (int k = 0; k < g; ++k) {
      sg_m0[k] = (int8_t)m;
      const int b = sg_e0[k];
      for (int e = b; e < sg_e0[k + 1]; ++e) end_row[e] = -1;
      for (int r = sg_row0[k]; r < sg_row0[k + 1]; ++r) {
        const VDesc d = rdesc[r];
        if (d.p == d.q && d.cp == 0 && d.cq == 0 && end_row[b + ip[r]] < 0)
          end_row[b + ip[r]] = (int16_t)r;
        else
          meta[m++] = make_int4(d.cp, d.cq, (int)ip[r] | ((int)iq[r] << 8), r);
      }
    }
    sg_m0[g] = (int8_t)m;
  }
  __syncthreads();
  if (tid < sg_e0[n_sg]) end_ptr[tid] = D + (int64_t)ends[tid] * ldd;
  __syncthreads();
  const int nsg = n_sg;
  const bool vec_ok = (ldo & 3) == 0;
  const uint32_t ldo_b = (uint32_t)(ldo * 4);
  int32_t *const oblk = out + (int64_t)(r0 - row_begin) * ldo;   // this CTA's first output row
  int32_t *Rw = R + w * 128;                                       // this warp's slice of every R row
  for (int32_t c0 = col_b + w * 128; c0 < col_e; c0 += CHUNK) {
    uint32_t op[4], oq[4];
    int32_t cpt[4], cqt[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int32_t t = c0 + 32 * j + lane;
      const VDesc d = t < n ? desc[t] : VDesc{0, 0, 0, 0};
      op[j] = (uint32_t)d.p * 4u; oq[j] = (uint32_t)d.q * 4u; cpt[j] = d.cp; cqt[j] = d.cq;
    }
    for (int g = 0; g < nsg; ++g) {
      const int e0 = sg_e0[g], ne = sg_e0[g + 1] - e0;
      for (int e = 0; e < ne; e += BATCH) {
        int32_t gp[BATCH][4], gq[BATCH][4];
#pragma unroll
        for (int u = 0; u < BATCH; ++u) {
          const int32_t *De = end_ptr[e0 + min(e + u, ne - 1)];   // past the last end: repeat it (cached)
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
            for (int j = 0; j < 4; ++j) {   // clamped to INF so that cp_s + R below cannot overflow
              v[j] = min(__viaddmin_s32(gq[u][j], cqt[j], gp[u][j] + cpt[j]), INF);
              Rw[(e + u) * CHUNK + 32 * j + lane] = v[j];
            }
            const int er = end_row[e0 + e + u];
            if (er >= 0) {   // warp-uniform: a terminal row of this sub-group -- emit it now
              int32_t *orow = row_ptr(oblk, er, ldo_b);
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
      if (ncol == 4 && vec_ok) {
        int last = -1;
        int4 a = make_int4(0, 0, 0, 0), b = a;
        for (int m = sg_m0[g]; m < m1; ++m) {
          const int4 md = meta[m];
          if (md.z != last) {   // consecutive rows of one chain share their R rows
            a = *reinterpret_cast<const int4 *>(Rw + (md.z & 0xFF) * CHUNK + lane * 4);
            b = *reinterpret_cast<const int4 *>(Rw + (md.z >> 8) * CHUNK + lane * 4);
            last = md.z;
          }
          int4 o;
          o.x = out_val(md.x, a.x, md.y, b.x);
          o.y = out_val(md.x, a.y, md.y, b.y);
          o.z = out_val(md.x, a.z, md.y, b.z);
          o.w = out_val(md.x, a.w, md.y, b.w);
          st_cs_v4(row_ptr(obase, md.w, ldo_b), o);
        }
      } else if (ncol > 0) {   // ragged tail or unaligned rows
        for (int m = sg_m0[g]; m < m1; ++m) {
          const int4 md = meta[m];
          const int32_t *ra = Rw + (md.z & 0xFF) * CHUNK + lane * 4, *rb = Rw + (md.z >> 8) * CHUNK + lane * 4;
          int32_t *orow = obase + (int64_t)md.w * ldo;
          for (int j = 0; j < ncol; ++j) orow[j] = out_val(md.x, ra[j], md.y, rb[j]);
        }
      }
      __syncwarp();
    }
  }
  __syncthreads();   // the next item rebuilds the shared row tables
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
__device__ __forceinline__ int32_t query_one(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc,
                                             const int32_t *__restrict__ ear, int32_t s, int32_t t) {
  const VDesc a = desc[s], b = desc[t];
  const int32_t *Dp = D + (int64_t)a.p * ldd, *Dq = D + (int64_t)a.q * ldd;
  // R[e,t] for e in {p_s, q_s} (2-term), then the 4-term rule
  const int32_t rp = min(__viaddmin_s32(Dp[b.q], b.cq, Dp[b.p] + b.cp), INF);
  const int32_t rq = min(__viaddmin_s32(Dq[b.q], b.cq, Dq[b.p] + b.cp), INF);
  int32_t v = min(__viaddmin_s32(a.cq, rq, a.cp + rp), INF);
  const int32_t es = ear[s];
  if (es >= 0 && es == ear[t]) v = min(v, abs(a.cp - b.cp));   // same chain (C8/C9)
  return v;
}
__global__ void k_query_pairs(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc,
                              const int32_t *__restrict__ ear, int64_t npairs, const int32_t *__restrict__ qs,
                              const int32_t *__restrict__ qt, int32_t *__restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < npairs; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = query_one(D, ldd, desc, ear, qs[i], qt[i]);
}

// Bucketed query: the pairs are first grouped by the source's left chain end p_s (a counting sort over
// the N_r terminals: histogram, scan, scatter of packed (s, t, i) records), so that the pairs of one
// bucket -- read consecutively -- share the D row p_s (and mostly q_s) while it sits in L2; the random
// D sectors of the per-pair kernel become L2 hits.  out[i] keeps the caller's pair order.
__global__ void k_qhist(int64_t npairs, const int32_t *__restrict__ qs, const VDesc *__restrict__ desc, int32_t *hist) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < npairs; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&hist[desc[qs[i]].p], 1);
}
__global__ void k_qscatter(int64_t npairs, const int32_t *__restrict__ qs, const int32_t *__restrict__ qt,
                           const VDesc *__restrict__ desc, int64_t *cur, int4 *rec) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < npairs; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t s = qs[i];
    const int64_t pos = atomicAdd(reinterpret_cast<unsigned long long *>(&cur[desc[s].p]), 1ull);
    rec[pos] = make_int4(s, qt[i], (int32_t)(i & 0xFFFFFFFF), (int32_t)(i >> 32));
  }
}
__global__ void k_query_bucketed(const int32_t *__restrict__ D, int64_t ldd, const VDesc *__restrict__ desc,
                                 const int32_t *__restrict__ ear, int64_t npairs, const int4 *__restrict__ rec,
                                 int32_t *__restrict__ out) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < npairs; j += (int64_t)gridDim.x * blockDim.x) {
    const int4 r = rec[j];
    out[(int64_t)(uint32_t)r.z | ((int64_t)r.w << 32)] = query_one(D, ldd, desc, ear, r.x, r.y);
  }
}
__global__ void k_hist64(int32_t nb, const int32_t *hist, int64_t *h64) {
  for (int32_t b = blockIdx.x * blockDim.x + threadIdx.x; b < nb; b += gridDim.x * blockDim.x) h64[b] = hist[b];
}


}  // namespace

ear_status_t expand(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t row_begin, int32_t row_end,
                    int32_t *out, int64_t ldo, cudaStream_t st, int prof_kind) {
  const int32_t rows = row_end - row_begin;
  if (rows <= 0) return EAR_OK;
  EAR_CUDA_TRY(smem_attr((const void *)k_expand, EXP_SMEM));
  int per = 0;
  EAR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_expand, NT, EXP_SMEM));
  const int32_t slots = std::max(1, num_sms() * std::max(per, 1));   // resident CTAs: one persistent wave
  const int32_t groups = (int32_t)ceil_div(rows, RB);
  ExpandWork W{};
  W.seg_w = (int32_t)round_up(ceil_div(plan->n, 8), CHUNK);
  W.nseg = (int32_t)ceil_div(plan->n, W.seg_w);
  const int32_t nsplit = std::min(groups, slots);
  W.n_full = groups - nsplit;
  W.n_items = W.n_full + nsplit * W.nseg;
  EAR_CUDA_TRY(cudaMallocAsync((void **)&W.counter, sizeof(int32_t), st));
  EAR_CUDA_TRY(dev_memset(W.counter, 0, sizeof(int32_t), st));
  const unsigned grid = (unsigned)std::min<int64_t>(W.n_items, slots);
  const double nr = plan->n_reduced;
  int se = prof_begin(prof_kind, st);
  EAR_LAUNCH(k_expand, grid, NT, EXP_SMEM, st)(D, ldd, plan->desc, plan->n, row_begin, row_end, out, ldo, W);
  prof_end(se, st, 4.0 * rows * plan->n + 16.0 * plan->n + 4.0 * nr * nr * rows / plan->n);
  if (plan->n_chain_vertices > 0) {
    int ss = prof_begin(prof_kind == PK_EXPAND ? PK_SAME_CHAIN : prof_kind, st);
    const int g2 = (int)std::min<int64_t>(ceil_div((int64_t)rows * 32, 256), 148 * 16);
    EAR_LAUNCH(k_same_chain, g2, 256, 0, st)(plan->desc, plan->seg_of, plan->seg_start, plan->seg_vert, row_begin,
                                      row_end, out, ldo);
    prof_end(ss, st, 0);
  }
  cudaFreeAsync(W.counter, st);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// Bucketing pays once a batch has many pairs per terminal row (EAR_QUERY_BUCKET_MIN overrides the
// threshold; 0 disables bucketing).
ear_status_t query_pairs(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int64_t npairs, const int32_t *qs,
                         const int32_t *qt, int32_t *out, cudaStream_t st) {
  if (npairs <= 0) return EAR_OK;
  const int grid = (int)std::min<int64_t>(ceil_div(npairs, 256), 148 * 16);
  const char *env = getenv("EAR_QUERY_BUCKET_MIN");
  const int64_t min_pairs = env ? atoll(env) : (int64_t)4 * plan->n_reduced + (1 << 20);
  if (min_pairs <= 0 || npairs < min_pairs) {
    EAR_LAUNCH(k_query_pairs, grid, 256, 0, st)(D, ldd, plan->desc, plan->ear, npairs, qs, qt, out);
    EAR_CUDA_TRY(cudaGetLastError());
    return EAR_OK;
  }
  const int32_t nb = std::max(plan->n_reduced, 1);
  int32_t *hist = nullptr;
  int64_t *h64 = nullptr, *start = nullptr;
  int4 *rec = nullptr;
  void *tmp = nullptr;
  size_t tb = 0;
  EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb, h64, start, nb, st));
  ear_status_t s = EAR_OK;
  if (cudaMallocAsync((void **)&hist, sizeof(int32_t) * nb, st) != cudaSuccess ||
      cudaMallocAsync((void **)&h64, sizeof(int64_t) * nb, st) != cudaSuccess ||
      cudaMallocAsync((void **)&start, sizeof(int64_t) * nb, st) != cudaSuccess ||
      cudaMallocAsync(&tmp, std::max<size_t>(tb, 16), st) != cudaSuccess ||
      cudaMallocAsync((void **)&rec, sizeof(int4) * (size_t)npairs, st) != cudaSuccess) {
    cudaGetLastError();
    s = EAR_ENOMEM;
    set_error("ear_query_pairs: out of device memory for the buckets");
  }
  if (s == EAR_OK) {
    const int gb = (int)std::min<int64_t>(ceil_div(nb, 256), 148 * 16);
    EAR_CUDA_TRY(dev_memset(hist, 0, sizeof(int32_t) * nb, st));
    EAR_LAUNCH(k_qhist, grid, 256, 0, st)(npairs, qs, plan->desc, hist);
    EAR_LAUNCH(k_hist64, gb, 256, 0, st)(nb, hist, h64);
    EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb, h64, start, nb, st));
    EAR_LAUNCH(k_qscatter, grid, 256, 0, st)(npairs, qs, qt, plan->desc, start, rec);
    EAR_LAUNCH(k_query_bucketed, grid, 256, 0, st)(D, ldd, plan->desc, plan->ear, npairs, rec, out);
  }
  for (void *p : {(void *)hist, (void *)h64, (void *)start, tmp, (void *)rec})
    if (p) cudaFreeAsync(p, st);
  EAR_TRY(s);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

}  // namespace ear
