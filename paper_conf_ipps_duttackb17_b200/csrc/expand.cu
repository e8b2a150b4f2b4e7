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
#include <mutex>
#include <vector>
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

__device__ __forceinline__ void st_cs_s32(int32_t *p, int32_t v) {
  asm volatile("st.global.cs.s32 [%0], %1;\n" ::"l"(p), "r"(v) : "memory");
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

// ============================================================================ pair-major expansion
// An item is one terminal v of G^r: its own output row (R[v, t], the 2-term rule seen from t)
// and the rows of every chain vertex s whose chain ends at v and at a partner x >= v (tid order; x = v
// for a closed ear): S[s, t] = min(c_sv + R[v, t], c_sx + R[x, t]) (the 4-term rule).  The D rows
// of v and of up to gcap partners are staged in shared memory as u16 (values < 0xFFFF, 0xFFFF = INF), so
// every D access is a shared-memory load; the column descriptors stream from L2 as packed 8-byte
// records; the output rows go out as 128-bit streaming stores.  No global gather is left, so the kernel
// is bound by the output stream, not by gather latency (the row-group kernel above), and it does not
// depend on how the caller labels the vertices.  Applies when N_r < 65535, every descriptor offset
// < 65536, every finite D entry < 0xFFFF and two u16 rows fit in shared memory; the same-chain clause
// is the separate k_same_chain pass as before.
constexpr int XP_NT = 1024;
constexpr int XP_RMAX = 64;   // chain rows written per column sweep
constexpr int XP_GMAX = 4;    // partner rows resident per sweep

struct XpView {
  const uint2 *pd;
  const int32_t *rows, *pstart, *px, *istart, *tid2v;
};

__global__ void k_xp_flags(int32_t n, const VDesc *desc, int32_t *bad) {
  int b = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const VDesc d = desc[v];
    b |= d.cp > 0xFFFF || d.cq > 0xFFFF || d.p > 0xFFFE || d.q > 0xFFFE;
  }
  if (__syncthreads_or(b) && threadIdx.x == 0) atomicOr(bad, 1);
}
__global__ void k_xp_desc(int32_t n, const VDesc *desc, uint2 *pd) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const VDesc d = desc[v];
    pd[v] = make_uint2((uint32_t)d.p | ((uint32_t)d.q << 16), (uint32_t)d.cp | ((uint32_t)d.cq << 16));
  }
}
__global__ void k_xp_keys(int32_t nc, const int32_t *seg_vert, const VDesc *desc, uint64_t *key, int32_t *val) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nc; i += gridDim.x * blockDim.x) {
    const int32_t v = seg_vert[i];
    const VDesc d = desc[v];
    key[i] = ((uint64_t)(uint32_t)min(d.p, d.q) << 32) | (uint32_t)max(d.p, d.q);
    val[i] = v;
  }
}
__global__ void k_xp_heads(int32_t nc, const uint64_t *key, int32_t *head) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nc; i += gridDim.x * blockDim.x)
    head[i] = i == 0 || key[i] != key[i - 1];
}
__global__ void k_xp_pairs(int32_t nc, const uint64_t *key, const int32_t *head, const int32_t *hscan, int32_t *pstart,
                           int32_t *px, int32_t *pcount) {
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nc; i += gridDim.x * blockDim.x)
    if (head[i]) {
      const int32_t j = hscan[i] - 1;
      pstart[j] = i;
      px[j] = (int32_t)(key[i] & 0xFFFFFFFFu);
      atomicAdd(&pcount[(int32_t)(key[i] >> 32)], 1);
    }
}
__global__ void k_xp_last(int32_t np, int32_t nc, int32_t *pstart) { pstart[np] = nc; }
__global__ void k_xp_last_dev(const int32_t *np, int32_t nc, int32_t *pstart) { pstart[*np] = nc; }
__global__ void k_xp_tid2v(int32_t n, const int32_t *tid, int32_t *tid2v) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    if (tid[v] >= 0) tid2v[tid[v]] = (int32_t)v;
}
// Label locality for the choice of expansion variant: one warp per sampled window of 32 consecutive
// columns; the window counts when its chain ends p_t (low half of pd.x) span fewer than XP_LOC_SPAN ids
// (one L1 line of 64 u16 per 32 lanes on average at the limit).  Morton labels: cfg4 87 %, cfg2 95 %;
// random labels: 0 %.
constexpr int XP_LOC_SAMPLES = 1024, XP_LOC_SPAN = 1024;
__global__ void k_xp_locality(const uint2 *__restrict__ pd, int32_t n, int32_t S, int32_t *count) {
  const int lane = threadIdx.x & 31;
  const int32_t w = (int32_t)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
  if (w >= S) return;
  const int32_t c = (int32_t)((int64_t)w * (n - 32) / S) + lane;
  const int32_t x = (int32_t)(pd[c].x & 0xFFFFu);
  int32_t lo = x, hi = x;
  for (int o = 16; o; o >>= 1) {
    lo = min(lo, __shfl_xor_sync(0xFFFFFFFFu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xFFFFFFFFu, hi, o));
  }
  if (lane == 0 && hi - lo < XP_LOC_SPAN) atomicAdd(count, 1);
}

// D (int32) -> u16 rows of stride ldr; a finite entry >= 0xFFFF sets *bad
__global__ void k_xp_d16(const int32_t *__restrict__ D, int64_t ldd, int32_t nr, int32_t ldr, uint16_t *__restrict__ D16,
                         int32_t *bad) {
  const int64_t total = (int64_t)nr * (ldr / 4);
  int b = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / (ldr / 4);
    const int32_t c = (int32_t)(i % (ldr / 4)) * 4;
    int32_t x[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int32_t v = c + k < nr ? D[r * ldd + c + k] : INF;
      b |= v >= 0xFFFF && v < INF;
      x[k] = v >= INF ? 0xFFFF : min(v, 0xFFFF);
    }
    *reinterpret_cast<uint2 *>(D16 + r * ldr + c) =
        make_uint2((uint32_t)x[0] | ((uint32_t)x[1] << 16), (uint32_t)x[2] | ((uint32_t)x[3] << 16));
  }
  if (__syncthreads_or(b) && threadIdx.x == 0) atomicOr(bad, 1);
}

// L2 prefetch of one D16 row (bytes: a multiple of 16), spread over the 32 lanes of a warp in 4 KB pieces
__device__ __forceinline__ void l2_prefetch_row(const uint16_t *row, int32_t bytes, int lane) {
  for (int32_t o = lane * 4096; o < bytes; o += 32 * 4096) {
    const int32_t sz = min(4096, bytes - o);
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;\n" ::"l"(reinterpret_cast<const char *>(row) + o), "r"(sz)
                 : "memory");
  }
}

__device__ __forceinline__ int32_t d16(const uint16_t *row, uint32_t t) {
  const uint32_t x = row[t];
  return x == 0xFFFFu ? INF : (int32_t)x;
}
// R[j] = min(D[row, p_t] + cp_t, D[row, q_t] + cq_t) for the 4 columns; CONN: G^r is connected, so no
// entry of D is INF (0xFFFF) and no clamping is needed
template <bool CONN>
__device__ __forceinline__ void r_of(const uint16_t *row, const uint32_t pq[4], const uint32_t cc[4], int32_t R[4]) {
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    if (CONN)
      R[j] = __viaddmin_s32((int32_t)row[pq[j] >> 16], (int32_t)(cc[j] >> 16),
                            (int32_t)row[pq[j] & 0xFFFFu] + (int32_t)(cc[j] & 0xFFFFu));
    else
      R[j] = min(__viaddmin_s32(d16(row, pq[j] >> 16), (int32_t)(cc[j] >> 16),
                                d16(row, pq[j] & 0xFFFFu) + (int32_t)(cc[j] & 0xFFFFu)), INF);
  }
}
// r_of over a row in global memory, read through the non-coherent path (D16 is read-only here)
template <bool CONN>
__device__ __forceinline__ void r_of_g(const uint16_t *row, const uint32_t pq[4], const uint32_t cc[4], int32_t R[4]) {
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint32_t a = __ldg(row + (pq[j] >> 16)), b = __ldg(row + (pq[j] & 0xFFFFu));
    if (CONN)
      R[j] = __viaddmin_s32((int32_t)a, (int32_t)(cc[j] >> 16), (int32_t)b + (int32_t)(cc[j] & 0xFFFFu));
    else
      R[j] = min(__viaddmin_s32(a == 0xFFFFu ? INF : (int32_t)a, (int32_t)(cc[j] >> 16),
                                (b == 0xFFFFu ? INF : (int32_t)b) + (int32_t)(cc[j] & 0xFFFFu)), INF);
  }
}
template <bool CONN>
__device__ __forceinline__ int32_t out_v(int32_t cp, int32_t rp, int32_t cq, int32_t rq) {
  return CONN ? __viaddmin_s32(cq, rq, cp + rp) : out_val(cp, rp, cq, rq);
}

// GP (global partners): only the item's row is staged; the partners' rows are gathered from D16 in
// global memory (L2-resident while the sweep runs), up to gcap = XP_GMAX of them per sweep.  With one row
// per CTA two 512-thread CTAs share an SM (cfg4: 60 KB rows), so one's sweep building and row staging
// overlap the other's column loop (measured 8.87 -> 8.47 ms on cfg4); rows too long for two per SM
// (cfg5: 120 KB) run one 1024-thread CTA per SM.  !GP: the partners' rows staged beside the item's.
template <bool CONN, bool GP, int NTT, bool LC = false>
__global__ void __launch_bounds__(NTT, 1024 / NTT)
    k_expand_pairs(const uint16_t *__restrict__ D16, int32_t ldr, int32_t nr, const VDesc *__restrict__ desc,
                   const XpView X, int32_t n, int32_t rb, int32_t re, int32_t *__restrict__ out, int64_t ldo,
                   int32_t gcap, int32_t *counter, int32_t pf) {
  extern __shared__ __align__(16) uint16_t srow[];   // [1 + gcap][ldr]
  __shared__ int4 meta[XP_RMAX];                     // {c_sv, c_sx, slot, local output row}
  __shared__ int4 runs[XP_RMAX];                     // {slot, first meta row, end}: one per pair in the sweep
  __shared__ int32_t slot_x[XP_GMAX];
  __shared__ int32_t s_item, s_nrow, s_ns, s_pj, s_rj, s_nrun;
  const int tid = threadIdx.x;
  const uint32_t ldo_b = (uint32_t)(ldo * 4);
  const int32_t row_bytes = ((nr + 7) / 8) * 16;
  for (;;) {
    if (tid == 0) s_item = atomicAdd(counter, 1);
    __syncthreads();
    const int32_t v = s_item;
    if (v >= nr) break;
    const int32_t tv = X.tid2v[v];
    bool need_term = tv >= rb && tv < re;
    const int32_t pe = X.istart[v + 1];
    int32_t pj = X.istart[v], rj = pj < pe ? X.pstart[pj] : 0;
    bool loaded_v = false;
    for (;;) {
      if (tid < 32) {   // warp 0 builds the next sweep: up to gcap partner rows, XP_RMAX chain rows in range
        const int lane = tid;
        int ns = 0, nrow = 0, nrun = 0;   // warp-uniform
        while (pj < pe && nrow < XP_RMAX) {
          const int32_t x = X.px[pj];
          int slot = 0;
          if (x != v) {
            slot = -1;
            for (int k = 0; k < ns; ++k)
              if (slot_x[k] == x) slot = k + 1;
            if (slot < 0) {
              if (ns == gcap) break;
              if (lane == 0) slot_x[ns] = x;
              if (GP && (pf & 1)) l2_prefetch_row(D16 + (int64_t)x * ldr, row_bytes, lane);
              __syncwarp();   // the other lanes read slot_x in the next partner's lookup
              slot = ++ns;
            }
          }
          const int32_t r1 = X.pstart[pj + 1];
          const int m0 = nrow;
          while (rj < r1 && nrow < XP_RMAX) {   // 32 rows of the pair at a time
            const int32_t idx = rj + lane;
            bool in = false;
            int4 mm = make_int4(0, 0, 0, 0);
            if (idx < r1) {
              const int32_t srow = X.rows[idx];
              in = srow >= rb && srow < re;
              if (in) {
                const VDesc d = desc[srow];
                const bool left = d.p == v;   // c_sv: along-chain distance from s to v
                mm = make_int4(left ? d.cp : d.cq, left ? d.cq : d.cp, slot, srow - rb);
              }
            }
            const unsigned bal = __ballot_sync(0xFFFFFFFFu, in);
            const int cap = XP_RMAX - nrow, cnt = __popc(bal);
            const int pos = __popc(bal & ((1u << lane) - 1u));
            if (in && pos < cap) meta[nrow + pos] = mm;
            if (cnt <= cap) {
              rj = min(r1, rj + 32);
              nrow += cnt;
            } else {   // full: resume right after the cap-th row in range
              unsigned b = bal;
              for (int q = 0; q < cap - 1; ++q) b &= b - 1u;
              rj += __ffs(b);
              nrow = XP_RMAX;
            }
          }
          if (nrow > m0) {
            if (lane == 0) runs[nrun] = make_int4(slot, m0, nrow, 0);
            ++nrun;
          }
          if (rj >= r1) {
            ++pj;
            if (pj < pe) rj = X.pstart[pj];
          }
        }
        __syncwarp();
        if (lane == 0) { s_nrow = nrow; s_ns = ns; s_pj = pj; s_rj = rj; s_nrun = nrun; }
      }
      __syncthreads();
      const int nrow = s_nrow, ns = s_ns, nrun = s_nrun;
      pj = s_pj;
      rj = s_rj;
      if (nrow > 0 || need_term) {
        const int nv = (nr + 7) / 8;   // 16-byte vectors per row
        if (!loaded_v)
          for (int i = tid; i < nv; i += NTT)
            reinterpret_cast<uint4 *>(srow)[i] = reinterpret_cast<const uint4 *>(D16 + (int64_t)v * ldr)[i];
        if (!GP)
          for (int k = 0; k < ns; ++k)
            for (int i = tid; i < nv; i += NTT)
              reinterpret_cast<uint4 *>(srow + (1 + k) * ldr)[i] =
                  reinterpret_cast<const uint4 *>(D16 + (int64_t)slot_x[k] * ldr)[i];
        loaded_v = true;
        __syncthreads();
        if constexpr (LC) {
          // lane-consecutive columns: lane l of warp w takes columns g*G + w*128 + l + 32*j (j < 4), so one
          // gather instruction of a warp covers 32 adjacent columns, whose chain ends are close together
          // (fewer distinct L1 lines / banks per gather than 4 columns per lane spread over 128)
          constexpr int32_t G = NTT * 4;
          const int32_t cw = (tid >> 5) * 128 + (tid & 31);
          uint2 nd[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) nd[j] = cw + 32 * j < n ? X.pd[cw + 32 * j] : make_uint2(0, 0);
          for (int32_t c0 = cw; c0 < n; c0 += G) {
            uint32_t pq[4], cc[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) { pq[j] = nd[j].x; cc[j] = nd[j].y; }
#pragma unroll
            for (int j = 0; j < 4; ++j) nd[j] = c0 + G + 32 * j < n ? X.pd[c0 + G + 32 * j] : make_uint2(0, 0);
            const bool full = c0 + 96 < n;
            int32_t Rv[4];
            r_of<CONN>(srow, pq, cc, Rv);
            if (need_term) {
              int32_t *o = reinterpret_cast<int32_t *>(reinterpret_cast<char *>(out) + (uint64_t)(uint32_t)(tv - rb) * ldo_b) + c0;
#pragma unroll
              for (int j = 0; j < 4; ++j)
                if (full || c0 + 32 * j < n) st_cs_s32(o + 32 * j, Rv[j]);
            }
            for (int ru = 0; ru < nrun; ++ru) {
              const int4 R = runs[ru];
              int32_t Rx[4];
              if (R.x == 0) {
#pragma unroll
                for (int j = 0; j < 4; ++j) Rx[j] = Rv[j];
              } else {
                const uint16_t *prow = D16 + (int64_t)slot_x[R.x - 1] * ldr;
                asm("" : "+l"(prow));   // one row pointer, not the row offset folded into every gather
                r_of_g<CONN>(prow, pq, cc, Rx);
              }
              for (int r = R.y; r < R.z; ++r) {
                const int4 m = meta[r];
                int32_t *o = reinterpret_cast<int32_t *>(reinterpret_cast<char *>(out) + (uint64_t)(uint32_t)m.w * ldo_b) + c0;
#pragma unroll
                for (int j = 0; j < 4; ++j)
                  if (full || c0 + 32 * j < n) st_cs_s32(o + 32 * j, out_v<CONN>(m.x, Rv[j], m.y, Rx[j]));
              }
            }
          }
          need_term = false;
        } else {
        // descriptors of the next column group are loaded while the current one is computed and stored
        uint4 na = make_uint4(0, 0, 0, 0), nb4 = make_uint4(0, 0, 0, 0);
        if (tid * 4 + 4 <= n) {
          na = *reinterpret_cast<const uint4 *>(X.pd + tid * 4);
          nb4 = *reinterpret_cast<const uint4 *>(X.pd + tid * 4 + 2);
        }
        for (int32_t c0 = tid * 4; c0 < n; c0 += NTT * 4) {
          uint32_t pq[4], cc[4];
          const bool full = c0 + 4 <= n;
          if (full) {
            pq[0] = na.x; cc[0] = na.y; pq[1] = na.z; cc[1] = na.w; pq[2] = nb4.x; cc[2] = nb4.y; pq[3] = nb4.z; cc[3] = nb4.w;
          } else {
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const uint2 q = c0 + j < n ? X.pd[c0 + j] : make_uint2(0, 0);
              pq[j] = q.x; cc[j] = q.y;
            }
          }
          const int32_t c1 = c0 + NTT * 4;
          if (c1 + 4 <= n) {
            na = *reinterpret_cast<const uint4 *>(X.pd + c1);
            nb4 = *reinterpret_cast<const uint4 *>(X.pd + c1 + 2);
          }
          int32_t Rv[4];
          r_of<CONN>(srow, pq, cc, Rv);
          if (need_term) {
            int32_t *o = reinterpret_cast<int32_t *>(reinterpret_cast<char *>(out) + (uint64_t)(uint32_t)(tv - rb) * ldo_b) + c0;
            if (full) st_cs_v4(o, make_int4(Rv[0], Rv[1], Rv[2], Rv[3]));
            else for (int j = 0; c0 + j < n; ++j) o[j] = Rv[j];
          }
          for (int ru = 0; ru < nrun; ++ru) {
            const int4 R = runs[ru];
            int32_t Rx[4];
            if (R.x == 0) {
#pragma unroll
              for (int j = 0; j < 4; ++j) Rx[j] = Rv[j];
            } else {
              r_of<CONN>(GP ? D16 + (int64_t)slot_x[R.x - 1] * ldr : srow + R.x * ldr, pq, cc, Rx);
            }
            for (int r = R.y; r < R.z; ++r) {
              const int4 m = meta[r];
              int4 o4;
              o4.x = out_v<CONN>(m.x, Rv[0], m.y, Rx[0]);
              o4.y = out_v<CONN>(m.x, Rv[1], m.y, Rx[1]);
              o4.z = out_v<CONN>(m.x, Rv[2], m.y, Rx[2]);
              o4.w = out_v<CONN>(m.x, Rv[3], m.y, Rx[3]);
              int32_t *o = reinterpret_cast<int32_t *>(reinterpret_cast<char *>(out) + (uint64_t)(uint32_t)m.w * ldo_b) + c0;
              if (full) st_cs_v4(o, o4);
              else {
                const int32_t t4[4] = {o4.x, o4.y, o4.z, o4.w};
                for (int j = 0; c0 + j < n; ++j) o[j] = t4[j];
              }
            }
          }
        }
        need_term = false;
        }
      }
      __syncthreads();   // the next sweep rewrites meta, slot_x and the partner rows
      if (pj >= pe) break;
    }
  }
}

}  // namespace

}  // namespace ear

struct ear_xp_s {
  int32_t ok = 0;            // the pair-major layout applies to this plan
  int32_t npairs = 0, nc = 0;   // npairs: not read back (pstart / px are sized by nc)
  uint2 *pd = nullptr;       // [n] packed descriptors {p | q << 16, cp | cq << 16}
  int32_t *rows = nullptr;   // [nc] chain vertices sorted by (smaller end, larger end, chain, offset)
  int32_t *pstart = nullptr; // [npairs + 1]
  int32_t *px = nullptr;     // [npairs] the larger end (the partner)
  int32_t *istart = nullptr; // [N_r + 1] the pairs of each item (terminal = smaller end)
  int32_t *tid2v = nullptr;  // [N_r]
  // label locality (k_xp_locality): sampled 32-column windows whose chain ends p_t span < XP_LOC_SPAN ids;
  // written into pinned host memory, complete when loc_ev is
  int32_t *loc_h = nullptr, *loc_d = nullptr, loc_samples = 0;
  cudaEvent_t loc_ev = nullptr;
};

namespace ear {

namespace {
// 4-byte pinned host slots for the locality counts, from one portable pinned page allocated once per
// process (a cudaHostAlloc / cudaFreeHost per plan would cost a synchronisation per apsp_full call)
struct PinnedSlots {
  std::mutex mu;
  int32_t *base = nullptr;
  std::vector<int> free;
  bool failed = false;
};
PinnedSlots &pinned_slots() {
  static PinnedSlots s;
  return s;
}
int32_t *slot_get() {
  PinnedSlots &s = pinned_slots();
  std::lock_guard<std::mutex> lk(s.mu);
  if (!s.base && !s.failed) {
    if (cudaHostAlloc((void **)&s.base, 4096 * sizeof(int32_t), cudaHostAllocPortable) != cudaSuccess) {
      cudaGetLastError();
      s.base = nullptr;
      s.failed = true;
    } else {
      for (int i = 4095; i >= 0; --i) s.free.push_back(i);
    }
  }
  if (!s.base || s.free.empty()) return nullptr;
  const int i = s.free.back();
  s.free.pop_back();
  return s.base + i;
}
void slot_put(int32_t *p) {
  PinnedSlots &s = pinned_slots();
  std::lock_guard<std::mutex> lk(s.mu);
  s.free.push_back((int)(p - s.base));
}
}  // namespace

void xp_free(ear_xp_s *x, cudaStream_t st) {
  if (!x) return;
  for (void *p : {(void *)x->pd, (void *)x->rows, (void *)x->pstart, (void *)x->px, (void *)x->istart, (void *)x->tid2v,
                  (void *)x->loc_d})
    if (p) cudaFreeAsync(p, st);
  if (x->loc_ev) {
    cudaEventSynchronize(x->loc_ev);
    cudaEventDestroy(x->loc_ev);
  }
  if (x->loc_h) slot_put(x->loc_h);
  delete x;
}

namespace {
// the item lists of the pair-major expansion, once per plan
ear_status_t xp_build(ear_plan_s *p, cudaStream_t st) {
  ear_xp_s *x = new ear_xp_s;
  p->xp = x;
  const int32_t n = p->n, nr = p->n_reduced, nc = p->n_chain_vertices;
  if (nr >= 0xFFFF) return EAR_OK;   // x->ok stays 0: the row-group kernel serves this plan
  if (!xp_bounds_fit(p)) {   // the host bound is not enough: check the descriptors on the device
    int32_t *bad = nullptr;
    EAR_CUDA_TRY(cudaMallocAsync((void **)&bad, sizeof(int32_t), st));
    EAR_CUDA_TRY(dev_memset(bad, 0, sizeof(int32_t), st));
    EAR_LAUNCH(k_xp_flags, (int)std::min<int64_t>(ceil_div(n, 256), 148 * 16), 256, 0, st)(n, p->desc, bad);
    int32_t h_bad = 1;
    {
      Readback rb(st);
      EAR_CUDA_TRY(rb.get(&h_bad, bad, sizeof(int32_t)));
      EAR_CUDA_TRY(rb.sync());
    }
    cudaFreeAsync(bad, st);
    if (h_bad) return EAR_OK;
  }
  auto g = [](int64_t k) { return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(k, 256), 148 * 16)); };
  EAR_CUDA_TRY(cudaMallocAsync((void **)&x->pd, sizeof(uint2) * (size_t)std::max(n, 1), st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&x->tid2v, sizeof(int32_t) * (size_t)std::max(nr, 1), st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&x->istart, sizeof(int32_t) * ((size_t)nr + 1), st));
  EAR_LAUNCH(k_xp_desc, g(n), 256, 0, st)(n, p->desc, x->pd);
  EAR_LAUNCH(k_xp_tid2v, g(n), 256, 0, st)(n, p->tid, x->tid2v);
  if (n >= 64 && (x->loc_h = slot_get()) != nullptr) {
    x->loc_samples = (int32_t)std::min<int64_t>(XP_LOC_SAMPLES, n / 32);
    EAR_CUDA_TRY(cudaMallocAsync((void **)&x->loc_d, sizeof(int32_t), st));
    EAR_CUDA_TRY(dev_memset(x->loc_d, 0, sizeof(int32_t), st));
    EAR_LAUNCH(k_xp_locality, ceil_div(x->loc_samples, 8), 256, 0, st)(x->pd, n, x->loc_samples, x->loc_d);
    EAR_CUDA_TRY(cudaMemcpyAsync(x->loc_h, x->loc_d, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
    EAR_CUDA_TRY(cudaEventCreateWithFlags(&x->loc_ev, cudaEventDisableTiming));
    EAR_CUDA_TRY(cudaEventRecord(x->loc_ev, st));
  }
  x->nc = nc;
  uint64_t *k0 = nullptr, *k1 = nullptr;
  int32_t *v0 = nullptr, *head = nullptr, *hscan = nullptr, *pcount = nullptr;
  void *tmp = nullptr;
  size_t tb = 0, tb2 = 0, tb3 = 0;
  const size_t m = (size_t)std::max(nc, 1);
  EAR_CUDA_TRY(cudaMallocAsync((void **)&x->rows, sizeof(int32_t) * m, st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&k0, sizeof(uint64_t) * m, st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&k1, sizeof(uint64_t) * m, st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&v0, sizeof(int32_t) * m, st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&head, sizeof(int32_t) * m, st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&hscan, sizeof(int32_t) * m, st));
  EAR_CUDA_TRY(cudaMallocAsync((void **)&pcount, sizeof(int32_t) * ((size_t)nr + 1), st));
  EAR_CUDA_TRY(dev_memset(pcount, 0, sizeof(int32_t) * ((size_t)nr + 1), st));
  int32_t npairs = 0;
  if (nc > 0) {
    EAR_LAUNCH(k_xp_keys, g(nc), 256, 0, st)(nc, p->seg_vert, p->desc, k0, v0);
    cub::DoubleBuffer<uint64_t> dk(k0, k1);
    cub::DoubleBuffer<int32_t> dv(v0, x->rows);
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, nc, 0, 64, st));
    EAR_CUDA_TRY(cub::DeviceScan::InclusiveSum(nullptr, tb2, head, hscan, nc, st));
    EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb3, pcount, x->istart, nr + 1, st));
    EAR_CUDA_TRY(cudaMallocAsync(&tmp, std::max({tb, tb2, tb3, (size_t)16}), st));
    EAR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dv, nc, 0, 64, st));
    if (dv.Current() != x->rows) EAR_CUDA_TRY(dev_copy(x->rows, dv.Current(), sizeof(int32_t) * nc, st));
    EAR_LAUNCH(k_xp_heads, g(nc), 256, 0, st)(nc, dk.Current(), head);
    EAR_CUDA_TRY(cub::DeviceScan::InclusiveSum(tmp, tb2, head, hscan, nc, st));
    // pairs <= chain vertices: sized by nc, so no host round trip for the pair count
    EAR_CUDA_TRY(cudaMallocAsync((void **)&x->pstart, sizeof(int32_t) * ((size_t)nc + 1), st));
    EAR_CUDA_TRY(cudaMallocAsync((void **)&x->px, sizeof(int32_t) * (size_t)std::max(nc, 1), st));
    EAR_LAUNCH(k_xp_pairs, g(nc), 256, 0, st)(nc, dk.Current(), head, hscan, x->pstart, x->px, pcount);
    EAR_LAUNCH(k_xp_last_dev, 1, 1, 0, st)(hscan + nc - 1, nc, x->pstart);
    EAR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb3, pcount, x->istart, nr + 1, st));
  } else {
    EAR_CUDA_TRY(cudaMallocAsync((void **)&x->pstart, sizeof(int32_t), st));
    EAR_CUDA_TRY(cudaMallocAsync((void **)&x->px, sizeof(int32_t), st));
    EAR_CUDA_TRY(dev_memset(x->pstart, 0, sizeof(int32_t), st));
    EAR_CUDA_TRY(dev_memset(x->istart, 0, sizeof(int32_t) * ((size_t)nr + 1), st));
  }
  for (void *q : {(void *)k0, (void *)k1, (void *)v0, (void *)head, (void *)hscan, (void *)pcount, tmp})
    if (q) cudaFreeAsync(q, st);
  x->npairs = npairs;
  x->ok = 1;
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

// the item's own u16 row of D fits in a CTA's shared memory
bool xp_row_fits(int32_t nr) {
  int dev = 0, smax = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&smax, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return round_up(std::max(nr, 1), 8) * 2 <= (int64_t)smax - 4096;
}

// partner rows that fit in shared memory beside the item's own row (0: the pair-major layout does not fit)
int32_t xp_gcap(int32_t nr) {
  int dev = 0, smax = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&smax, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  const int64_t rowb = round_up(std::max(nr, 1), 8) * 2, budget = (int64_t)smax - 4096;
  return (int32_t)std::max<int64_t>(0, std::min<int64_t>(XP_GMAX, budget / rowb - 1));
}

// k_expand_pairs over u16 rows D16 (stride ld16) + the same-chain pass; the caller checked applicability
ear_status_t launch_pairs(const ear_plan_s *plan, const uint16_t *D16, int32_t ld16, int32_t row_begin, int32_t row_end,
                          int32_t *out, int64_t ldo, cudaStream_t st, int prof_kind) {
  NvtxRange nvtx_("ear: expansion (pair-major)");
  const ear_xp_s *x = plan->xp;
  const int32_t nr = plan->n_reduced;
  // GP with two 512-thread CTAs per SM when two single-row CTAs fit an SM's shared memory, GP with one
  // 1024-thread CTA when only one row fits beside nothing else, the partners staged otherwise (never: a
  // row that fits twice in a CTA fits twice in an SM).
  int dev = 0, per_sm = 0;
  EAR_CUDA_TRY(cudaGetDevice(&dev));
  EAR_CUDA_TRY(cudaDeviceGetAttribute(&per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev));
  const int64_t rowb = (int64_t)ld16 * 2;
  const char *force = getenv("EAR_XP_GP");   // tests: 0 staged partners, 1 global (two CTAs/SM), 2 global (one)
  const int fv = force ? atoi(force) : -1;
  const bool two = 2 * (rowb + 4096) <= per_sm && fv != 2;
  // labels without locality (random: every gather its own sector) make the partners' gathers the
  // bottleneck once D16 outgrows L2 (DRAM sectors): stage them instead when they fit (cfg4 random labels
  // 19.6 -> 11.6 ms, Morton 9.2 vs 9.5; cfg2 random, D16 in L2: 0.55 global vs 0.66 staged)
  bool local = true;
  int l2 = 0;
  EAR_CUDA_TRY(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev));
  if (x->loc_ev && (int64_t)nr * rowb > l2 && cudaEventSynchronize(x->loc_ev) == cudaSuccess)
    local = 2 * *x->loc_h >= x->loc_samples;
  const bool gp = fv >= 0 ? fv >= 1 : ((two && local) || xp_gcap(nr) < 1);
  int32_t gcap = gp ? XP_GMAX : xp_gcap(nr);
  if (const char *e = getenv("EAR_XP_GCAP")) gcap = std::max(1, std::min(gcap, atoi(e)));   // lab knob
  const char *le = getenv("EAR_XP_LC");   // lab knob: 0 = four adjacent columns per lane
  const bool lc = gp && (le ? atoi(le) != 0 : true);
  const int smem = (int)((gp ? 1 : 1 + gcap) * rowb);
  const char *pfe = getenv("EAR_XP_PF");
  const int32_t pf = pfe ? atoi(pfe) : 0;   // lab knob: 1 = the partners' rows prefetched into L2
  const bool conn = plan->connected == 1;
  const void *kf = lc ? (two ? (conn ? (const void *)k_expand_pairs<true, true, 512, true> : (const void *)k_expand_pairs<false, true, 512, true>)
                              : (conn ? (const void *)k_expand_pairs<true, true, 1024, true> : (const void *)k_expand_pairs<false, true, 1024, true>))
                 : gp ? (two ? (conn ? (const void *)k_expand_pairs<true, true, 512> : (const void *)k_expand_pairs<false, true, 512>)
                             : (conn ? (const void *)k_expand_pairs<true, true, 1024> : (const void *)k_expand_pairs<false, true, 1024>))
                      : (conn ? (const void *)k_expand_pairs<true, false, 1024> : (const void *)k_expand_pairs<false, false, 1024>);
  EAR_CUDA_TRY(smem_attr(kf, smem));
  int32_t *counter = nullptr;
  EAR_CUDA_TRY(cudaMallocAsync((void **)&counter, sizeof(int32_t), st));
  EAR_CUDA_TRY(dev_memset(counter, 0, sizeof(int32_t), st));
  const XpView V{x->pd, x->rows, x->pstart, x->px, x->istart, x->tid2v};
  const double rows = row_end - row_begin;
  int se = prof_begin(prof_kind, st);
#define XP_GO(C, G, T, B)                                                                                      \
  EAR_LAUNCH((k_expand_pairs<C, G, T>), (B) * num_sms(), T, smem, st)(D16, ld16, nr, plan->desc, V, plan->n, \
                                                                       row_begin, row_end, out, ldo, gcap, counter, pf)
#define XP_LC(C, T, B)                                                                                               \
  EAR_LAUNCH((k_expand_pairs<C, true, T, true>), (B) * num_sms(), T, smem, st)(D16, ld16, nr, plan->desc, V, plan->n, \
                                                                                row_begin, row_end, out, ldo, gcap, counter, pf)
  if (lc && two) {
    if (conn) XP_LC(true, 512, 2); else XP_LC(false, 512, 2);
  } else if (lc) {
    if (conn) XP_LC(true, 1024, 1); else XP_LC(false, 1024, 1);
  } else if (gp && two) {
    if (conn) XP_GO(true, true, 512, 2); else XP_GO(false, true, 512, 2);
  } else if (gp) {
    if (conn) XP_GO(true, true, 1024, 1); else XP_GO(false, true, 1024, 1);
  } else {
    if (conn) XP_GO(true, false, 1024, 1); else XP_GO(false, false, 1024, 1);
  }
#undef XP_GO
#undef XP_LC
  // algorithmic bytes: the output, D read once (counted as the int32 D, as for the row-group kernel), the
  // descriptors
  prof_end(se, st, 4.0 * rows * plan->n + 16.0 * plan->n + 4.0 * (double)nr * nr * rows / plan->n);
  cudaFreeAsync(counter, st);
  if (plan->n_chain_vertices > 0) {
    int ss = prof_begin(prof_kind == PK_EXPAND ? PK_SAME_CHAIN : prof_kind, st);
    const int g2 = (int)std::min<int64_t>(ceil_div((int64_t)(row_end - row_begin) * 32, 256), 148 * 16);
    EAR_LAUNCH(k_same_chain, g2, 256, 0, st)(plan->desc, plan->seg_of, plan->seg_start, plan->seg_vert, row_begin,
                                              row_end, out, ldo);
    prof_end(ss, st, 0);
  }
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

bool aligned_out(const int32_t *out, int64_t ldo) { return (ldo & 3) == 0 && (reinterpret_cast<uintptr_t>(out) & 15) == 0; }

// the pair-major expansion from the int32 D (narrowed to u16 rows first) when it applies: *done = true
// after writing the rows, the same-chain pass included
ear_status_t expand_pairs(ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t row_begin, int32_t row_end,
                          int32_t *out, int64_t ldo, cudaStream_t st, int prof_kind, bool *done) {
  *done = false;
  if (!aligned_out(out, ldo) || !xp_applicable(plan, st)) return EAR_OK;
  const int32_t nr = plan->n_reduced, ldr = xp_row_stride(plan);
  uint16_t *D16 = nullptr;
  int32_t *bad = nullptr;
  if (cudaMallocAsync((void **)&D16, sizeof(uint16_t) * (size_t)nr * ldr, st) != cudaSuccess ||
      cudaMallocAsync((void **)&bad, sizeof(int32_t), st) != cudaSuccess) {
    cudaGetLastError();
    if (D16) cudaFreeAsync(D16, st);
    return EAR_OK;
  }
  ear_status_t s = EAR_OK;
  int32_t h_bad = 1;
  {
    cudaError_t e = dev_memset(bad, 0, sizeof(int32_t), st);
    const int64_t tot = (int64_t)nr * (ldr / 4);
    int sp = prof_begin(prof_kind == PK_EXPAND ? PK_EXPAND_D16 : prof_kind, st);
    if (e == cudaSuccess && tot > 0)
      EAR_LAUNCH(k_xp_d16, (int)std::min<int64_t>(ceil_div(tot, 256), 148 * 16), 256, 0, st)(D, ldd, nr, ldr, D16, bad);
    prof_end(sp, st, 0);
    Readback rb(st);
    if (e == cudaSuccess) e = rb.get(&h_bad, bad, sizeof(int32_t));
    if (e == cudaSuccess) e = rb.sync();
    if (e != cudaSuccess) { set_error("expand: %s", cudaGetErrorString(e)); s = EAR_ECUDA; }
  }
  if (s == EAR_OK && !h_bad) {
    s = launch_pairs(plan, D16, ldr, row_begin, row_end, out, ldo, st, prof_kind);
    *done = s == EAR_OK;
  }
  cudaFreeAsync(D16, st);
  cudaFreeAsync(bad, st);
  return s;
}
}  // namespace

int32_t xp_row_stride(const ear_plan_s *plan) { return (int32_t)round_up(std::max(plan->n_reduced, 1), 8); }

// every chain offset fits 16 bits by the host's bound ((longest chain + 1) x heaviest edge) and every
// terminal id too: the item lists can be built without a device check (no host round trip)
bool xp_bounds_fit(const ear_plan_s *p) {
  return p->n_reduced < 0xFFFF && ((int64_t)p->max_chain_len + 1) * (int64_t)std::max(p->max_weight, 0) <= 0xFFFF;
}

// xp_applicable's answer known on the host without building anything: the lists exist and apply, or
// they will (no device check needed, the item's row fits a CTA)
bool xp_predict(const ear_plan_s *plan) {
  const char *env = getenv("EAR_EXPAND_PAIRS");
  if (env && atoi(env) == 0) return false;
  if (plan->xp) return plan->xp->ok != 0;
  return xp_bounds_fit(plan) && xp_row_fits(plan->n_reduced);
}

bool xp_applicable(ear_plan_s *plan, cudaStream_t st) {
  const char *env = getenv("EAR_EXPAND_PAIRS");   // 0: the row-group kernel (A/B)
  if (env && atoi(env) == 0) return false;
  // one row beside the item's (gcap >= 1), or -- partners then gathered from global memory -- the item's row alone
  if (plan->n_reduced >= 0xFFFF || !xp_row_fits(plan->n_reduced)) return false;
  if (!plan->xp && xp_build(plan, st) != EAR_OK) {
    cudaGetLastError();
    return false;
  }
  return plan->xp && plan->xp->ok;
}

ear_status_t expand_from16(const ear_plan_s *plan, const uint16_t *D16, int32_t ld16, int32_t row_begin, int32_t row_end,
                           int32_t *out, int64_t ldo, cudaStream_t st, int prof_kind) {
  if (row_end <= row_begin) return EAR_OK;
  if (!plan->xp || !plan->xp->ok || !aligned_out(out, ldo) || ld16 < xp_row_stride(plan)) {
    set_error("expand_from16: the pair-major layout does not apply");
    return EAR_EUNSUPPORTED;
  }
  return launch_pairs(plan, D16, ld16, row_begin, row_end, out, ldo, st, prof_kind);
}

ear_status_t expand(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int32_t row_begin, int32_t row_end,
                    int32_t *out, int64_t ldo, cudaStream_t st, int prof_kind) {
  const int32_t rows = row_end - row_begin;
  if (rows <= 0) return EAR_OK;
  if (prof_kind == PK_EXPAND) {   // the caller's rows; a BCC piece's re-expansion keeps the row-group kernel
    bool done = false;             // (its plan is built per solve: the item lists would be rebuilt each time)
    EAR_TRY(expand_pairs(const_cast<ear_plan_s *>(plan), D, ldd, row_begin, row_end, out, ldo, st, prof_kind, &done));
    if (done) return EAR_OK;
  }
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

// One thread per pair.  Measured on cfg4 (profiles/r02g_query_mode_cfg4.jsonl): 1.53e10 uniformly random
// pairs/s, 3.60e10 when the caller's pairs are grouped by source (1,024 targets per source: the D rows
// p_s, q_s stay in L2); an in-library counting sort of the pairs by p_s cost more than it saved (0.65x).
ear_status_t query_pairs(const ear_plan_s *plan, const int32_t *D, int64_t ldd, int64_t npairs, const int32_t *qs,
                         const int32_t *qt, int32_t *out, cudaStream_t st) {
  if (npairs <= 0) return EAR_OK;
  const int grid = (int)std::min<int64_t>(ceil_div(npairs, 256), 148 * 16);
  EAR_LAUNCH(k_query_pairs, grid, 256, 0, st)(D, ldd, plan->desc, plan->ear, npairs, qs, qt, out);
  EAR_CUDA_TRY(cudaGetLastError());
  return EAR_OK;
}

}  // namespace ear
