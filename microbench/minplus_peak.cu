// Int32 min-plus issue-rate microbenchmark for sm_100a (roofline denominator for the FW kernels).
// Each variant runs independent register-only chains of the form c_i = min(c_i, c_{i+1} + b)
// (not idempotent, so the compiler cannot fold repeats).  Reported: min-plus ops/s over the whole
// GPU, and ops/clk/SM over each SM's busy window -- from the first block start to the last block end
// on that SM, both read from the SM's own clock64 (round 1 divided by the mean per-BLOCK window, which
// undercounts cycles whenever blocks of an SM do not overlap exactly and gave inconsistent figures).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define NACC 16
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ int imad1(int a, int one, int b) {
  int r; asm volatile("mad.lo.s32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(one), "r"(b)); return r;
}

// variant 0: VIADDMNMX only (1 op / instr)
// variant 1: IMAD+IMAD (fma pipe) + VIMNMX3 (2 ops / 3 instr)
// variant 2: half of the accumulators variant 0, half variant 1
// variant 3: FADD + FMNMX (fp32 on integer values)
// variant 4: VIADDMNMX.S16x2 (2 ops / instr, 16-bit lanes)
// variant 5: VIADDMNMX.U16x2 (2 ops / instr, unsigned 16-bit lanes)
template <int V>
__global__ void __launch_bounds__(256) mp_kernel(int* out, const int* in, int iters, long long* cyc) {
  int c[NACC];
  int one = in[0];
  int b0 = in[1 + (threadIdx.x & 7)], b1 = in[2 + (threadIdx.x & 7)];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) c[i] = in[16 + ((threadIdx.x + i) & 63)];
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i) {
      if (V == 0) {
        c[i] = __viaddmin_s32(c[(i + 1) % NACC], b0, c[i]);
      } else if (V == 1) {
        int x = imad1(c[(i + 1) % NACC], one, b0);
        int y = imad1(c[(i + 2) % NACC], one, b1);
        c[i] = __vimin3_s32(c[i], x, y);
      } else if (V == 2) {
        if (i & 1) {
          int x = imad1(c[(i + 1) % NACC], one, b0);
          int y = imad1(c[(i + 2) % NACC], one, b1);
          c[i] = __vimin3_s32(c[i], x, y);
        } else {
          c[i] = __viaddmin_s32(c[(i + 1) % NACC], b0, c[i]);
        }
      } else if (V == 3) {
        float f = __int_as_float(c[(i + 1) % NACC]) + __int_as_float(b0);
        c[i] = __float_as_int(fminf(__int_as_float(c[i]), f));
      } else if (V == 4) {
        c[i] = __viaddmin_s16x2(c[(i + 1) % NACC], b0, c[i]);
      } else if (V == 5) {
        c[i] = __viaddmin_u16x2(c[(i + 1) % NACC], b0, c[i]);
      }
    }
  }
  long long t1 = clock64();
  int s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s ^= c[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    cyc[3 * blockIdx.x] = smid;
    cyc[3 * blockIdx.x + 1] = t0;
    cyc[3 * blockIdx.x + 2] = t1;
  }
}

template <int V>
int run(const char* name, double ops_per_update, int nsm, int* d_out, int* d_in, long long* d_cyc) {
  int threads = 256, blocks = nsm * 8, iters = 20000;
  mp_kernel<V><<<blocks, threads>>>(d_out, d_in, 100, d_cyc);
  CK(cudaDeviceSynchronize());
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e30f;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0);
    mp_kernel<V><<<blocks, threads>>>(d_out, d_in, iters, d_cyc);
    cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  static long long h_cyc[3 * 148 * 64];
  CK(cudaMemcpy(h_cyc, d_cyc, sizeof(long long) * 3 * blocks, cudaMemcpyDeviceToHost));
  // per SM: busy window = last end - first start on that SM's clock; ops of the blocks that ran there
  static long long lo[1024], hi[1024], nb[1024];
  for (int i = 0; i < 1024; ++i) { lo[i] = -1; hi[i] = 0; nb[i] = 0; }
  for (int b = 0; b < blocks; ++b) {
    const int sm = (int)h_cyc[3 * b];
    if (sm < 0 || sm >= 1024) continue;
    if (lo[sm] < 0 || h_cyc[3 * b + 1] < lo[sm]) lo[sm] = h_cyc[3 * b + 1];
    if (h_cyc[3 * b + 2] > hi[sm]) hi[sm] = h_cyc[3 * b + 2];
    nb[sm]++;
  }
  double updates = (double)blocks * threads * iters * NACC;
  double ops = updates * ops_per_update;
  double ratio = 0, win = 0;
  int used = 0;
  for (int sm = 0; sm < 1024; ++sm)
    if (nb[sm]) {
      const double w = (double)(hi[sm] - lo[sm]);
      ratio += (double)nb[sm] * threads * iters * NACC * ops_per_update / w;
      win += w;
      ++used;
    }
  double ops_per_clk_sm = ratio / used;           // mean over SMs of that SM's ops / its busy cycles
  double eff_mhz = (win / used) / (best * 1e-3) / 1e6;   // busy cycles per SM / kernel time
  printf("{\"variant\": \"%s\", \"ms\": %.3f, \"Tops_per_s\": %.3f, \"ops_per_clk_per_sm\": %.1f, \"eff_sm_mhz\": %.0f, "
         "\"sms_used\": %d, \"blocks\": %d}\n",
         name, best, ops / (best * 1e-3) / 1e12, ops_per_clk_sm, eff_mhz, used, blocks);
  return 0;
}

// semantics of the unsigned 16x2 add-min at the top of the range (wrap or saturate?)
__global__ void u16_semantics(unsigned *out) {
  const unsigned a[6] = {0x7FFF7FFFu, 0x80008000u, 0xFFFF0001u, 0xC0004000u, 0xFFFEFFFFu, 0x00050003u};
  const unsigned b[6] = {0x7FFF0001u, 0x80000001u, 0x0001FFFFu, 0x4000C000u, 0x00010001u, 0x00020004u};
  const unsigned c[6] = {0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0x00060006u};
  for (int i = 0; i < 6; ++i) out[i] = __viaddmin_u16x2(a[i], b[i], c[i]);
}

int main() {
  int dev = 0; cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  int nsm = p.multiProcessorCount;
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"cc\": \"%d.%d\"}\n", p.name, nsm, p.major, p.minor);
  int *d_out, *d_in; long long* d_cyc;
  CK(cudaMalloc(&d_out, sizeof(int) * nsm * 8 * 256));
  CK(cudaMalloc(&d_cyc, sizeof(long long) * 3 * nsm * 8));
  int h_in[128]; h_in[0] = 1; for (int i = 1; i < 128; ++i) h_in[i] = (i * 37) % 101 + 1;
  CK(cudaMalloc(&d_in, sizeof(h_in))); CK(cudaMemcpy(d_in, h_in, sizeof(h_in), cudaMemcpyHostToDevice));
  run<0>("viaddmnmx", 1.0, nsm, d_out, d_in, d_cyc);
  run<1>("imad2_vimnmx3", 1.0, nsm, d_out, d_in, d_cyc);
  run<2>("mixed_1to1", 1.0, nsm, d_out, d_in, d_cyc);
  run<3>("fadd_fmnmx", 1.0, nsm, d_out, d_in, d_cyc);
  run<4>("viaddmnmx_s16x2", 2.0, nsm, d_out, d_in, d_cyc);
  run<5>("viaddmnmx_u16x2", 2.0, nsm, d_out, d_in, d_cyc);
  {
    unsigned *d_s, h_s[6];
    CK(cudaMalloc(&d_s, sizeof(h_s)));
    u16_semantics<<<1, 1>>>(d_s);
    CK(cudaMemcpy(h_s, d_s, sizeof(h_s), cudaMemcpyDeviceToHost));
    printf("{\"u16x2_addmin\": [\"%08x\", \"%08x\", \"%08x\", \"%08x\", \"%08x\", \"%08x\"], "
           "\"inputs\": \"a+b min c for a=7fff7fff+7fff0001, 80008000+80000001, ffff0001+0001ffff, c0004000+4000c000, fffeffff+00010001, 00050003+00020004 (c=00060006)\"}\n",
           h_s[0], h_s[1], h_s[2], h_s[3], h_s[4], h_s[5]);
  }
  run<0>("viaddmnmx_again", 1.0, nsm, d_out, d_in, d_cyc);
  return 0;
}
