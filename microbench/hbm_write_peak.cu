// Store-only HBM bandwidth on the B200 (context for the expansion kernel's HBM roofline):
// a grid-stride kernel of 128-bit streaming stores (st.global.cs.v4) and cudaMemsetAsync, each over
// a 40 GB buffer (the cfg4 output size), best of 5, CUDA events.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_store(int4 *p, size_t n16, int v) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += stride) {
    int4 x = make_int4(v, v + 1, v + 2, (int)i);
    asm volatile("st.global.cs.v4.s32 [%0], {%1, %2, %3, %4};" ::"l"(p + i), "r"(x.x), "r"(x.y), "r"(x.z), "r"(x.w) : "memory");
  }
}

__global__ void k_store_plain(int4 *p, size_t n16, int v) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += stride) p[i] = make_int4(v, v, v, (int)i);
}

int main() {
  size_t bytes = 40ull << 30;
  void *buf;
  if (cudaMalloc(&buf, bytes) != cudaSuccess) { printf("{\"error\": \"alloc\"}\n"); return 1; }
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  auto bench = [&](const char *name, auto fn) {
    float best = 1e30f;
    for (int r = 0; r < 6; ++r) {
      cudaEventRecord(a); fn(r); cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b); if (r > 0 && ms < best) best = ms;
    }
    printf("{\"what\": \"%s\", \"bytes\": %zu, \"ms\": %.3f, \"GBps\": %.1f}\n", name, bytes, best, bytes / (best * 1e-3) / 1e9);
  };
  int sms = 148; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  bench("st.global.cs.v4 grid-stride (4 x 148 x 256 thr... 8 CTAs/SM)", [&](int r) { k_store<<<sms * 8, 256>>>((int4 *)buf, bytes / 16, r); });
  bench("plain int4 stores", [&](int r) { k_store_plain<<<sms * 8, 256>>>((int4 *)buf, bytes / 16, r); });
  bench("cudaMemsetAsync", [&](int r) { cudaMemsetAsync(buf, r, bytes); });
  return 0;
}
