#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <chrono>
#include <vector>
#include <algorithm>
typedef unsigned int u32; typedef unsigned long long u64;
__device__ __forceinline__ u64 gt() { u64 t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ u32 ldrel(const u32* p) { u32 v; asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p)); return v; }
__device__ __forceinline__ u32 ldsys(const u32* p) { u32 v; asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p)); return v; }
__global__ void spin(const u32* flag, u64* out, int sys) {
  u64 t0 = gt();
  if (sys) { while (ldsys(flag) == 0u) { if (gt() - t0 > 100000000ull) break; } }
  else { while (ldrel(flag) == 0u) { if (gt() - t0 > 100000000ull) break; } }
  if (threadIdx.x == 0) { out[0] = t0; out[1] = gt(); }
}
int main() {
  u32* flag; u64* out; cudaMalloc(&flag, 256); cudaMalloc(&out, 64);
  u32 *hflag, *hone; cudaHostAlloc(&hflag, 64, cudaHostAllocMapped); cudaHostAlloc(&hone, 64, 0); *hone = 1;
  u32* dflag_host; cudaHostGetDevicePointer(&dflag_host, hflag, 0);
  cudaStream_t a, nb; cudaStreamCreateWithFlags(&a, cudaStreamNonBlocking); cudaStreamCreateWithFlags(&nb, cudaStreamNonBlocking);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const char* names[] = {"memop (default)", "memop NO_MEMORY_BARRIER", "memcpyAsync pinned H2D", "host store to mapped pinned flag (ld.sys)"};
  for (int variant = 0; variant < 4; variant++) {
    std::vector<double> ev, host;
    for (int t = 0; t < 30; t++) {
      cudaMemset(flag, 0, 4); *hflag = 0; cudaDeviceSynchronize();
      spin<<<1, 32, 0, a>>>(variant == 3 ? dflag_host : flag, out, variant == 3);
      cudaEventRecord(e1, a);
      auto t0 = std::chrono::steady_clock::now();
      while (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() < 3e-4) {}
      cudaEventRecord(e0, nb);
      auto th0 = std::chrono::steady_clock::now();
      if (variant == 0) cuStreamWriteValue32((CUstream)nb, (CUdeviceptr)flag, 1, 0);
      else if (variant == 1) cuStreamWriteValue32((CUstream)nb, (CUdeviceptr)flag, 1, CU_STREAM_WRITE_VALUE_NO_MEMORY_BARRIER);
      else if (variant == 2) cudaMemcpyAsync(flag, hone, 4, cudaMemcpyHostToDevice, nb);
      else { __atomic_store_n(hflag, 1u, __ATOMIC_SEQ_CST); }
      cudaStreamSynchronize(a);
      auto th1 = std::chrono::steady_clock::now();
      cudaStreamSynchronize(nb);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      ev.push_back(ms * 1e3); host.push_back(std::chrono::duration<double, std::micro>(th1 - th0).count());
    }
    std::sort(ev.begin(), ev.end()); std::sort(host.begin(), host.end());
    printf("%-44s event p50 %.2f us p90 %.2f | host issue->spinner done p50 %.2f us p90 %.2f\n", names[variant], ev[15], ev[27], host[15], host[27]);
  }
}
