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

// TMA bulk stores (cp.async.bulk.global.shared::cta) from a shared-memory staging buffer: each warp
// streams CHUNK-byte pieces of its contiguous part of the buffer, NBUF staging slots deep.
template <int CHUNK, int NBUF>
__global__ void k_store_bulk(char *p, size_t bytes, int v) {
  extern __shared__ __align__(128) char sbuf[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  char *mine = sbuf + (size_t)w * NBUF * CHUNK;
  for (int i = lane; i < NBUF * CHUNK / 16; i += 32)
    reinterpret_cast<int4 *>(mine)[i] = make_int4(v, v, v, i);
  __syncwarp();
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  const size_t nchunks = bytes / CHUNK;
  const size_t gw = (size_t)blockIdx.x * nw + w, nwarps = (size_t)gridDim.x * nw;
  int slot = 0;
  for (size_t c = gw; c < nchunks; c += nwarps) {
    if (lane == 0) {
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(p + c * CHUNK),
                   "r"((uint32_t)__cvta_generic_to_shared(mine + slot * CHUNK)), "r"(CHUNK) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(NBUF - 1) : "memory");
    }
    slot = (slot + 1) % NBUF;
  }
  if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
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
  cudaFuncSetAttribute(k_store_bulk<4096, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 4 * 4096);
  bench("TMA bulk store 4 KB pieces, 4 slots/warp, 8 warps x 148 x 1 CTA", [&](int r) {
    k_store_bulk<4096, 4><<<sms, 256, 8 * 4 * 4096>>>((char *)buf, bytes, r); });
  cudaFuncSetAttribute(k_store_bulk<512, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16 * 8 * 512);
  bench("TMA bulk store 512 B pieces, 8 slots/warp, 16 warps x 148 x 2 CTAs", [&](int r) {
    k_store_bulk<512, 8><<<sms * 2, 512, 16 * 8 * 512>>>((char *)buf, bytes, r); });
  cudaFuncSetAttribute(k_store_bulk<2048, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 4 * 2048);
  bench("TMA bulk store 2 KB pieces, 4 slots/warp, 8 warps x 148 x 2 CTAs", [&](int r) {
    k_store_bulk<2048, 4><<<sms * 2, 256, 8 * 4 * 2048>>>((char *)buf, bytes, r); });
  printf("{\"error_check\": \"%s\"}\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
