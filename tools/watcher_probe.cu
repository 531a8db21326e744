// How fast can a device warp notice a store to mapped pinned host memory?
// Host: store seq to the host word, spin until the device acks (a system-scope
// store to another host word) -> round trip = detection + ack write.
// Variants of the watcher's polling loop:
//   0: one warp, one outstanding system-scope load at a time (CTXB_WATCHER)
//   1: one warp, 4 loads in flight (software-pipelined, each lane group its own)
//   2: 4 watcher warps on different SMs, each one load at a time
//   3: one warp, ld.volatile.sys (weak) instead of ld.relaxed.sys
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/watcher_probe tools/watcher_probe.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <vector>
typedef unsigned int u32;

__device__ __forceinline__ u32 ld_sys(const volatile u32* p) {
  u32 v; asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ u32 ld_vol(const volatile u32* p) {
  u32 v; asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ void st_sys(volatile u32* p, u32 v) {
  asm volatile("st.relaxed.sys.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory"); }

template <int V>
__global__ void watch(const volatile u32* hw, volatile u32* ack, u32 rounds) {
  const u32 lane = threadIdx.x & 31u;
  for (u32 r = 1; r <= rounds; r++) {
    if (V == 1) {
      // four independent loads in flight; a lane group per slot
      u32 a = ld_sys(hw), b = ld_sys(hw), c = ld_sys(hw), d = ld_sys(hw);
      while (a < r && b < r && c < r && d < r) {
        a = b; b = c; c = d; d = ld_sys(hw);
      }
    } else if (V == 3) {
      while (ld_vol(hw) < r) {}
    } else {
      while (ld_sys(hw) < r) {}
    }
    if (lane == 0 && (V != 2 || blockIdx.x == 0)) st_sys(ack, r);
    if (V == 2) { while (ld_sys(ack) < r) {} }   // keep the four in step
  }
}

int main() {
  u32 *hw, *ack, *dhw, *dack;
  cudaHostAlloc(&hw, 64, cudaHostAllocMapped);
  cudaHostAlloc(&ack, 64, cudaHostAllocMapped);
  cudaHostGetDevicePointer(&dhw, hw, 0);
  cudaHostGetDevicePointer(&dack, ack, 0);
  const char* names[] = {"1 warp, 1 load in flight (relaxed.sys)", "1 warp, 4 loads in flight",
                         "4 warps (4 SMs), 1 load each", "1 warp, ld.volatile"};
  const u32 rounds = 200;
  for (int v = 0; v < 4; v++) {
    *(volatile u32*)hw = 0; *(volatile u32*)ack = 0;
    cudaStream_t s; cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    if (v == 0) watch<0><<<1, 32, 0, s>>>(dhw, dack, rounds);
    if (v == 1) watch<1><<<1, 32, 0, s>>>(dhw, dack, rounds);
    if (v == 2) watch<2><<<4, 32, 0, s>>>(dhw, dack, rounds);
    if (v == 3) watch<3><<<1, 32, 0, s>>>(dhw, dack, rounds);
    std::vector<double> rt;
    auto spin = [](double us) { auto t = std::chrono::steady_clock::now();
      while (std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t).count() < us) {} };
    spin(20000);
    for (u32 r = 1; r <= rounds; r++) {
      spin(37.0 + (r % 7));           // desynchronise from the device's read cadence
      auto t0 = std::chrono::steady_clock::now();
      *(volatile u32*)hw = r;
      while (*(volatile u32*)ack < r) {}
      rt.push_back(std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count());
    }
    cudaStreamSynchronize(s);
    std::sort(rt.begin(), rt.end());
    printf("%-40s host store -> device ack: p10 %.2f p50 %.2f p90 %.2f us\n", names[v], rt[rt.size() / 10],
           rt[rt.size() / 2], rt[rt.size() * 9 / 10]);
    cudaStreamDestroy(s);
  }
  return 0;
}
