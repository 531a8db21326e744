// Preemption-signal paths, second probe (B200): does stream priority or the
// memop flavour change the flag's propagation time?  A one-warp spinner polls
// a device flag with ld.relaxed.gpu; the control stream records an event and
// then raises the flag; elapsed = that event -> an event after the spinner
// (upper bound: includes the spinner's exit).  Every API return code is
// checked.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -o probe2 signal_probe2.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <vector>
typedef unsigned int u32;
typedef unsigned long long u64;
#define CK(x) do { auto e_ = (x); if (e_ != 0) { printf("  %s -> error %d\n", #x, (int)e_); return -1; } } while (0)
__device__ __forceinline__ u64 gt() { u64 t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ u32 ldrel(const u32* p) { u32 v; asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p)); return v; }
__global__ void spin(const u32* flag, u64* out) {
  u64 t0 = gt();
  while (ldrel(flag) == 0u) { if (gt() - t0 > 20000000ull) break; }
  if (threadIdx.x == 0) { out[0] = t0; out[1] = gt(); }
}
__global__ void setflag(u32* flag) { if (threadIdx.x == 0) asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" :: "l"(flag), "r"(1u)); }

static int trial(const char* name, int variant, int prio) {
  u32* flag; u64* out;
  CK(cudaMalloc(&flag, 256)); CK(cudaMalloc(&out, 64));
  cudaStream_t a, nb;
  CK(cudaStreamCreateWithFlags(&a, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithPriority(&nb, cudaStreamNonBlocking, prio));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  std::vector<double> ev, host; int timeouts = 0;
  for (int t = 0; t < 40; t++) {
    CK(cudaMemset(flag, 0, 4)); CK(cudaDeviceSynchronize());
    spin<<<1, 32, 0, a>>>(flag, out);
    CK(cudaEventRecord(e1, a));
    auto t0 = std::chrono::steady_clock::now();
    while (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() < 3e-4) {}
    CK(cudaEventRecord(e0, nb));
    auto th0 = std::chrono::steady_clock::now();
    if (variant == 0) CK(cuStreamWriteValue32((CUstream)nb, (CUdeviceptr)flag, 1, 0));
    else if (variant == 1) CK(cuStreamWriteValue32((CUstream)nb, (CUdeviceptr)flag, 1, CU_STREAM_WRITE_VALUE_NO_MEMORY_BARRIER));
    else if (variant == 2) {
      CUstreamBatchMemOpParams p = {};
      p.writeValue.operation = CU_STREAM_MEM_OP_WRITE_VALUE_32;
      p.writeValue.address = (CUdeviceptr)flag;
      p.writeValue.value = 1;
      p.writeValue.flags = 0;
      CK(cuStreamBatchMemOp((CUstream)nb, 1, &p, 0));
    } else if (variant == 3) {
      setflag<<<1, 32, 0, nb>>>(flag);
      CK(cudaGetLastError());
    }
    CK(cudaStreamSynchronize(a));
    auto th1 = std::chrono::steady_clock::now();
    CK(cudaStreamSynchronize(nb));
    u64 h[2]; CK(cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost));
    if (h[1] - h[0] > 19000000ull) timeouts++;
    float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
    ev.push_back(ms * 1e3); host.push_back(std::chrono::duration<double, std::micro>(th1 - th0).count());
  }
  std::sort(ev.begin(), ev.end()); std::sort(host.begin(), host.end());
  printf("%-44s prio %2d: event p50 %6.2f p90 %6.2f us | host issue->spinner done p50 %6.2f us | timeouts %d\n", name, prio,
         ev[20], ev[36], host[20], timeouts);
  cudaStreamDestroy(a); cudaStreamDestroy(nb); cudaFree(flag); cudaFree(out);
  return 0;
}

int main() {
  int lo, hi; cudaDeviceGetStreamPriorityRange(&lo, &hi);
  printf("stream priority range: least %d greatest %d\n", lo, hi);
  const char* names[] = {"cuStreamWriteValue32 (default)", "cuStreamWriteValue32 NO_MEMORY_BARRIER",
                         "cuStreamBatchMemOp write32", "1-thread kernel st.relaxed.gpu (idle GPU only)"};
  for (int v = 0; v < 4; v++)
    for (int pr : {lo, hi}) trial(names[v], v, pr);
  return 0;
}
