// Probe: two processes on ONE GPU exchange data through CUDA IPC peer mappings (the transport of the
// sharded FW's per-round exchange).  Each process allocates a window, sends its IPC handle to the
// other over a pipe, opens the peer's window, writes a block into it with a kernel, publishes a flag
// with a system-scope release, waits for the peer's flag (spin kernel, and cuStreamWaitValue32 when the
// device supports it) and checks the data it received.  Prints one JSON line per process.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o ipc_probe ipc_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <sys/wait.h>
#include <unistd.h>

#include <chrono>
#include <cstdio>
#include <cstring>

#define CK(x)                                                                              \
  do {                                                                                     \
    cudaError_t e = (x);                                                                   \
    if (e != cudaSuccess) {                                                                \
      printf("{\"rank\": %d, \"error\": \"%s: %s\"}\n", rank, #x, cudaGetErrorString(e)); \
      return 1;                                                                            \
    }                                                                                      \
  } while (0)

constexpr size_t kWords = 1 << 20;   // 4 MB payload

__global__ void k_put(unsigned *peer_data, unsigned long long *peer_flag, unsigned tag, unsigned long long val) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < kWords; i += (size_t)gridDim.x * blockDim.x)
    peer_data[i] = tag ^ (unsigned)i;
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) {
    // every block bumps the peer's flag; the peer waits for gridDim.x * val
    asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(peer_flag), "l"(val) : "memory");
  }
}

__global__ void k_wait(const unsigned long long *flag, unsigned long long target) {
  unsigned long long v = 0;
  do {
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(flag) : "memory");
  } while (v < target);
}

__global__ void k_check(const unsigned *data, unsigned tag, int *bad) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < kWords; i += (size_t)gridDim.x * blockDim.x)
    if (data[i] != (tag ^ (unsigned)i)) atomicAdd(bad, 1);
}

int run(int rank, int wfd, int rfd) {
  CK(cudaSetDevice(0));
  char *win = nullptr;
  const size_t bytes = kWords * 4 + 256;
  CK(cudaMalloc(&win, bytes));
  CK(cudaMemset(win, 0, bytes));
  CK(cudaDeviceSynchronize());
  cudaIpcMemHandle_t mine, theirs;
  CK(cudaIpcGetMemHandle(&mine, win));
  if (write(wfd, &mine, sizeof(mine)) != (ssize_t)sizeof(mine)) return 2;
  if (read(rfd, &theirs, sizeof(theirs)) != (ssize_t)sizeof(theirs)) return 2;
  char *peer = nullptr;
  CK(cudaIpcOpenMemHandle((void **)&peer, theirs, cudaIpcMemLazyEnablePeerAccess));
  unsigned *my_data = (unsigned *)win, *peer_data = (unsigned *)peer;
  unsigned long long *my_flag = (unsigned long long *)(win + kWords * 4);
  unsigned long long *peer_flag = (unsigned long long *)(peer + kWords * 4);
  int *bad = nullptr;
  CK(cudaMalloc(&bad, 4));
  CK(cudaMemset(bad, 0, 4));
  cudaStream_t st;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  const int grid = 64;
  auto t0 = std::chrono::steady_clock::now();
  // round 1: spin-kernel wait
  k_put<<<grid, 256, 0, st>>>(peer_data, peer_flag, 0xA5000000u | rank, 1);
  k_wait<<<1, 1, 0, st>>>(my_flag, grid);
  k_check<<<grid, 256, 0, st>>>(my_data, 0xA5000000u | (1 - rank), bad);
  CK(cudaStreamSynchronize(st));
  auto t1 = std::chrono::steady_clock::now();
  int h_bad = -1;
  CK(cudaMemcpy(&h_bad, bad, 4, cudaMemcpyDeviceToHost));
  // round 2: cuStreamWaitValue64 (front-end wait, no SM) when supported
  int can_wait = 0;
  cudaDeviceGetAttribute(&can_wait, (cudaDeviceAttr)CU_DEVICE_ATTRIBUTE_CAN_USE_STREAM_WAIT_VALUE_NOR, 0);
  int mem_ops = -1;
  {
    CUdevice d;
    cuInit(0);
    cuDeviceGet(&d, 0);
    cuDeviceGetAttribute(&mem_ops, CU_DEVICE_ATTRIBUTE_CAN_USE_64_BIT_STREAM_MEM_OPS, d);
  }
  int bad2 = -1;
  double ms2 = -1;
  const char *wv = "untried";
  {
    CK(cudaMemset(bad, 0, 4));
    CK(cudaDeviceSynchronize());
    auto t2 = std::chrono::steady_clock::now();
    k_put<<<grid, 256, 0, st>>>(peer_data, peer_flag, 0x5A000000u | rank, 1);
    CUresult r = cuStreamWaitValue64((CUstream)st, (CUdeviceptr)my_flag, (cuuint64_t)(2 * grid), CU_STREAM_WAIT_VALUE_GEQ);
    if (r != CUDA_SUCCESS) {
      wv = "cuStreamWaitValue64 failed; spin fallback";
      k_wait<<<1, 1, 0, st>>>(my_flag, 2 * grid);
    } else {
      wv = "cuStreamWaitValue64 ok";
    }
    k_check<<<grid, 256, 0, st>>>(my_data, 0x5A000000u | (1 - rank), bad);
    CK(cudaStreamSynchronize(st));
    ms2 = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t2).count();
    CK(cudaMemcpy(&bad2, bad, 4, cudaMemcpyDeviceToHost));
  }
  printf("{\"rank\": %d, \"spin_bad\": %d, \"spin_ms\": %.3f, \"waitvalue\": \"%s\", \"waitvalue_bad\": %d, "
         "\"waitvalue_ms\": %.3f, \"attr_wait_nor\": %d, \"attr_64bit_memops\": %d}\n",
         rank, h_bad, std::chrono::duration<double, std::milli>(t1 - t0).count(), wv, bad2, ms2, can_wait, mem_ops);
  fflush(stdout);
  cudaIpcCloseMemHandle(peer);
  return 0;
}

int main() {
  int a[2], b[2];
  if (pipe(a) || pipe(b)) return 3;
  pid_t pid = fork();
  int rank = pid == 0 ? 1 : 0;
  int rc = rank == 0 ? run(0, a[1], b[0]) : run(1, b[1], a[0]);
  if (rank == 1) _exit(rc);
  int st = 0;
  waitpid(pid, &st, 0);
  return rc | WEXITSTATUS(st);
}
