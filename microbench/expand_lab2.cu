// Expansion lab, round 2: template variants of the library's k_expand (csrc/expand.cu) on the same
// items, sub-groups and R tiles -- AHEAD: exact-address L2 prefetch (prefetch.global.L2::evict_last) of
// every gather of the chunk AHEAD chunks ahead, for all ends of the item; EVL: gathers with an
// L2::evict_last cache policy (D outlives the streamed output in L2); D16: gathers from a u16 copy of D
// (0xFFFF = INF).  lab2_expand(variant, ...) runs one; tools/expand_lab2.py times them bit-exactly.
#include <algorithm>
#include <cstdlib>

#include "common.cuh"

namespace ear {
namespace {
constexpr int NT = 256;
constexpr int RB = 32;
constexpr int ECAP = 16;
constexpr int CHUNK = 1024;
constexpr int BATCH = 4;
#define EXP_MINB 2
constexpr int EXP_SMEM = ECAP * CHUNK * 4;

template <int D16> struct DTs { using T = int32_t; };
template <> struct DTs<1> { using T = uint16_t; };
template <int D16> using DT = typename DTs<D16>::T;

__device__ __forceinline__ void st_cs_v4(int32_t *p, int4 v) {
  asm volatile("st.global.cs.v4.s32 [%0], {%1, %2, %3, %4};\n" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}
__device__ __forceinline__ int32_t out_val(int32_t cp, int32_t rp, int32_t cq, int32_t rq) {
  return min(__viaddmin_s32(cq, rq, cp + rp), INF);
}
template <int EVL, int D16>
__device__ __forceinline__ int32_t gat(const DT<D16> *base, uint32_t byte_off, uint64_t pol) {
  const char *p = reinterpret_cast<const char *>(base) + byte_off;
  if (D16) {
    uint16_t v;
    if (EVL) asm volatile("ld.global.nc.L2::cache_hint.u16 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol));
    else v = __ldg(reinterpret_cast<const uint16_t *>(p));
    return v == 0xFFFFu ? INF : (int32_t)v;
  }
  int32_t v;
  if (EVL) asm volatile("ld.global.nc.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  else v = __ldg(reinterpret_cast<const int32_t *>(p));
  return v;
}
__device__ __forceinline__ int32_t *row_ptr(int32_t *base, int32_t r, uint32_t ld_bytes) {
  return reinterpret_cast<int32_t *>(reinterpret_cast<char *>(base) + (uint64_t)(uint32_t)r * ld_bytes);
}
struct ExpandWork {
  int32_t *counter;
  int32_t n_full, n_items, nseg, seg_w;
};
template <int AHEAD, int EVL, int D16>
__global__ void __launch_bounds__(NT, EXP_MINB) k_expand_v(const DT<D16> *__restrict__ D, int64_t ldd,
                                                 const VDesc *__restrict__ desc, int32_t n, int32_t row_begin,
                                                 int32_t row_end, int32_t *__restrict__ out, int64_t ldo,
                                                 const ExpandWork W) {
  extern __shared__ __align__(16) int32_t R[];       // [ECAP][CHUNK]
  __shared__ VDesc rdesc[RB];
  __shared__ int32_t ends[2 * RB];                   // endpoint tids, sub-group by sub-group
  __shared__ const DT<D16> *end_ptr[2 * RB];         // their D rows
  __shared__ int16_t end_row[2 * RB];                // local output row of a terminal end in its sub-group, or -1
  __shared__ int8_t ip[RB], iq[RB];                  // per row: index of p / q in its sub-group
  __shared__ int8_t sg_row0[RB + 1], sg_e0[RB + 1];  // sub-group g: rows [row0[g], row0[g+1]), ends [e0[g], e0[g+1])
  __shared__ int4 meta[RB];                          // chain rows by sub-group: {cp, cq, ip | iq << 8, local row}
  __shared__ int8_t sg_m0[RB + 1];
  __shared__ int32_t n_sg, item_sh;

  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  uint64_t pol = 0;
  if (EVL) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
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
      op[j] = (uint32_t)d.p * (uint32_t)sizeof(DT<D16>); oq[j] = (uint32_t)d.q * (uint32_t)sizeof(DT<D16>);
      cpt[j] = d.cp; cqt[j] = d.cq;
    }
    if (AHEAD > 0) {   // exact-address L2 prefetch of the gathers of chunk + AHEAD (all ends of the item)
      const int32_t cn = c0 + AHEAD * CHUNK;
      if (cn < col_e) {
        const int ntot = sg_e0[nsg];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int32_t t = cn + 32 * j + lane;
          if (t < n) {
            const VDesc d = desc[t];
            const uint32_t a = (uint32_t)d.p * (uint32_t)sizeof(DT<D16>), b = (uint32_t)d.q * (uint32_t)sizeof(DT<D16>);
            for (int e = 0; e < ntot; ++e) {
              const char *base = reinterpret_cast<const char *>(end_ptr[e]);
              asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(base + a));
              if (b != a) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(base + b));
            }
          }
        }
      }
    }
    for (int g = 0; g < nsg; ++g) {
      const int e0 = sg_e0[g], ne = sg_e0[g + 1] - e0;
      for (int e = 0; e < ne; e += BATCH) {
        int32_t gp[BATCH][4], gq[BATCH][4];
#pragma unroll
        for (int u = 0; u < BATCH; ++u) {
          const DT<D16> *De = end_ptr[e0 + min(e + u, ne - 1)];   // past the last end: repeat it (cached)
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            gp[u][j] = gat<EVL, D16>(De, op[j], pol);
            gq[u][j] = gat<EVL, D16>(De, oq[j], pol);
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


template <int AHEAD, int EVL, int D16>
int run(const ear_plan_s *plan, const void *D, int64_t ldd, int32_t rb, int32_t re, int32_t *out, int64_t ldo,
        cudaStream_t st) {
  auto k = k_expand_v<AHEAD, EVL, D16>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, EXP_SMEM);
  int per = 0, sms = 0, dev = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k, NT, EXP_SMEM);
  const int32_t slots = std::max(1, sms * std::max(per, 1));
  const int32_t rows = re - rb, groups = (rows + RB - 1) / RB;
  ExpandWork W{};
  W.seg_w = (int32_t)(((plan->n + 7) / 8 + CHUNK - 1) / CHUNK * CHUNK);
  W.nseg = (plan->n + W.seg_w - 1) / W.seg_w;
  const int32_t nsplit = std::min(groups, slots);
  W.n_full = groups - nsplit;
  W.n_items = W.n_full + nsplit * W.nseg;
  cudaMallocAsync((void **)&W.counter, 4, st);
  cudaMemsetAsync(W.counter, 0, 4, st);
  k<<<std::min(W.n_items, slots), NT, EXP_SMEM, st>>>((const DT<D16> *)D, ldd, plan->desc, plan->n, rb, re, out, ldo, W);
  cudaFreeAsync(W.counter, st);
  return cudaGetLastError() == cudaSuccess ? 0 : 1;
}
}  // namespace
}  // namespace ear

// variants: 1 = prefetch 1 ahead, 2 = prefetch 2 ahead, 3 = evict_last gathers, 4 = u16 D,
// 5 = u16 D + prefetch 1, 6 = prefetch 1 + evict_last, 7 = u16 D + prefetch 2, 10 = baseline copy
extern "C" int lab2_expand(int variant, const ear_plan_s *plan, const void *D, int64_t ldd, int32_t rb, int32_t re,
                           int32_t *out, int64_t ldo, void *stream) {
  using namespace ear;
  cudaStream_t st = (cudaStream_t)stream;
  switch (variant) {
    case 1: return run<1, 0, 0>(plan, D, ldd, rb, re, out, ldo, st);
    case 2: return run<2, 0, 0>(plan, D, ldd, rb, re, out, ldo, st);
    case 3: return run<0, 1, 0>(plan, D, ldd, rb, re, out, ldo, st);
    case 4: return run<0, 0, 1>(plan, D, ldd, rb, re, out, ldo, st);
    case 5: return run<1, 0, 1>(plan, D, ldd, rb, re, out, ldo, st);
    case 6: return run<1, 1, 0>(plan, D, ldd, rb, re, out, ldo, st);
    case 7: return run<2, 0, 1>(plan, D, ldd, rb, re, out, ldo, st);
    case 10: return run<0, 0, 0>(plan, D, ldd, rb, re, out, ldo, st);
  }
  return 2;
}
