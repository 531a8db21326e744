// Micro-benchmark: how fast can 2368 resident warps (296 blocks x 256 threads,
// C2's persistent grid) read their own L2-cold context slot of `slot` bytes
// (C2 CTXBack: 8844 B per warp = 20.9 MB) into registers?  Span = max over
// warps of t_done - min over warps of t_start (%globaltimer), like the resume
// time.  Variants:
//   0 ldg      : 16 B per lane per 512 B group, ld.global.cs.v4 (the restore stub)
//   1 hdr+ldg  : a dependent 16 B header load first (the resume dispatch)
//   2 tma      : lane 0 issues cp.async.bulk global->shared for the warp's slot
//                (mbarrier complete_tx), then every lane reads its values
//                from shared memory
//   3 hdr+tma  : header load, then 2
//   4 ldg.nc   : ld.global.nc.L2::256B.v4
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/restore_micro tools/restore_micro.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

typedef unsigned int u32;
typedef unsigned long long u64;

__device__ __forceinline__ u64 gt() { u64 t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }

template <int V>
__global__ void __launch_bounds__(256, 2) rd(const unsigned char* ctx, const uint4* hdr, u32 slot, u32 zero,
                                             u64* st, u32* out) {
  extern __shared__ __align__(128) unsigned char sm[];
  const u32 lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  const u32 gw = blockIdx.x * 8 + warp;
  const u64 t0 = gt();
  const unsigned char* pay = ctx + (u64)gw * slot;
  u32 acc = 0;
  u32 ng = slot / 512;
  if (V == 1 || V == 3) {
    uint4 h = __ldcg(hdr + gw);
    acc ^= h.x;
    if ((h.x & zero) != 0u) return;   // dependent: payload issued after the header returned
    pay += (h.y & zero);
  }
  if (V == 0 || V == 1) {
#pragma unroll 1
    for (u32 g = 0; g < ng; g += 8) {
      uint4 q[8];
#pragma unroll
      for (int j = 0; j < 8; j++)
        if (g + j < ng) q[j] = __ldcs(reinterpret_cast<const uint4*>(pay + (g + j) * 512) + lane);
#pragma unroll
      for (int j = 0; j < 8; j++)
        if (g + j < ng) acc ^= q[j].x ^ q[j].y ^ q[j].z ^ q[j].w;
    }
  } else if (V == 4) {
#pragma unroll 1
    for (u32 g = 0; g < ng; g += 8) {
      uint4 q[8];
#pragma unroll
      for (int j = 0; j < 8; j++)
        if (g + j < ng)
          asm volatile("ld.global.nc.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
                       : "=r"(q[j].x), "=r"(q[j].y), "=r"(q[j].z), "=r"(q[j].w)
                       : "l"(reinterpret_cast<const uint4*>(pay + (g + j) * 512) + lane));
#pragma unroll
      for (int j = 0; j < 8; j++)
        if (g + j < ng) acc ^= q[j].x ^ q[j].y ^ q[j].z ^ q[j].w;
    }
  } else {
    __shared__ __align__(8) u64 bar[8];
    unsigned char* dst = sm + warp * slot;
    u32 sbar = (u32)__cvta_generic_to_shared(&bar[warp]);
    u32 sdst = (u32)__cvta_generic_to_shared(dst);
    if (lane == 0) {
      asm volatile("mbarrier.init.shared.b64 [%0], 1;" :: "r"(sbar));
      asm volatile("fence.mbarrier_init.release.cluster;");
      asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" :: "r"(sbar), "r"(slot));
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   :: "r"(sdst), "l"(pay), "r"(slot), "r"(sbar) : "memory");
    }
    __syncwarp();
    u32 done = 0;
    while (!done)
      asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                   : "=r"(done) : "r"(sbar) : "memory");
    for (u32 g = 0; g < ng; g++) {
      uint4 q = reinterpret_cast<const uint4*>(dst + g * 512)[lane];
      acc ^= q.x ^ q.y ^ q.z ^ q.w;
    }
  }
  acc = __reduce_xor_sync(0xffffffffu, acc);
  u64 t1 = 0;
  if ((acc & zero) == 0u) t1 = gt();
  if (lane == 0) { st[gw * 2] = t0; st[gw * 2 + 1] = t1; out[gw] = acc; }
}

int main(int argc, char** argv) {
  const u32 slot = argc > 1 ? (u32)atoi(argv[1]) : 8704;   // multiple of 512
  const int blocks = argc > 2 ? atoi(argv[2]) : 296;
  const int reps = 9;
  const u32 nw = blocks * 8;
  unsigned char* ctx; uint4* hdr; u64* st; u32* out; int* scr;
  cudaMalloc(&ctx, (size_t)nw * slot);
  cudaMalloc(&hdr, nw * 16);
  cudaMalloc(&st, nw * 16);
  cudaMalloc(&out, nw * 4);
  cudaMalloc(&scr, 256u << 20);
  cudaMemset(ctx, 1, (size_t)nw * slot);
  cudaMemset(hdr, 0, nw * 16);
  const char* names[] = {"ldg", "hdr+ldg", "tma", "hdr+tma", "ldg.nc.L2::256B"};
  void (*ks[])(const unsigned char*, const uint4*, u32, u32, u64*, u32*) = {rd<0>, rd<1>, rd<2>, rd<3>, rd<4>};
  for (int v = 0; v < 5; v++) {
    size_t smem = (v == 2 || v == 3) ? (size_t)8 * slot : 0;
    if (smem) cudaFuncSetAttribute(ks[v], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    std::vector<double> span;
    for (int r = 0; r < reps + 1; r++) {
      cudaMemset(scr, r, 256u << 20);     // evict L2
      ks[v]<<<blocks, 256, smem>>>(ctx, hdr, slot, 0u, st, out);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("%s: %s\n", names[v], cudaGetErrorString(e)); return 1; }
      std::vector<u64> h(nw * 2);
      cudaMemcpy(h.data(), st, nw * 16, cudaMemcpyDeviceToHost);
      u64 a = ~0ull, b = 0;
      for (u32 w = 0; w < nw; w++) { a = std::min(a, h[w * 2]); b = std::max(b, h[w * 2 + 1]); }
      if (r) span.push_back((b - a) / 1e3);
    }
    std::sort(span.begin(), span.end());
    double med = span[span.size() / 2];
    printf("%-16s slot %u B x %u warps = %.1f MB: span p50 %.2f us (min %.2f) -> %.0f GB/s\n", names[v], slot, nw,
           nw * (double)slot / 1e6, med, span[0], nw * (double)slot / med / 1e3);
  }
  return 0;
}
