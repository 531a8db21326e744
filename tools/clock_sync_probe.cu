// Host-clock <-> %globaltimer offset on the GPU box, NTP style: the host
// writes k to a mapped pinned word (time h1, CLOCK_REALTIME), a one-thread
// kernel spinning on it stamps %globaltimer (g) and acknowledges through
// another mapped word, the host sees the ack (h2).  offset = g - (h1 + h2)/2,
// uncertain by +-(h2 - h1)/2; the minimum-RTT sample is printed.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o tools/clock_sync_probe tools/clock_sync_probe.cu
#include <cstdio>
#include <ctime>
#include <cuda_runtime.h>

__global__ void spin(volatile unsigned* in, volatile unsigned* ack, unsigned long long* g, unsigned n) {
  for (unsigned k = 1; k <= n; k++) {
    unsigned v;
    do { asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(in)); } while (v != k);
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g[k] = t;
    __threadfence_system();
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;" :: "l"(ack), "r"(k) : "memory");
  }
}

static long long now_ns() {
  timespec ts;
  clock_gettime(CLOCK_REALTIME, &ts);
  return (long long)ts.tv_sec * 1000000000LL + ts.tv_nsec;
}

int main() {
  const unsigned n = 200;
  unsigned *in, *ack;
  unsigned long long* g;
  cudaHostAlloc(&in, 64, cudaHostAllocMapped);
  cudaHostAlloc(&ack, 64, cudaHostAllocMapped);
  cudaHostAlloc(&g, (n + 1) * 8, cudaHostAllocMapped);
  *in = 0; *ack = 0;
  unsigned *din, *dack;
  unsigned long long* dg;
  cudaHostGetDevicePointer(&din, in, 0);
  cudaHostGetDevicePointer(&dack, ack, 0);
  cudaHostGetDevicePointer(&dg, g, 0);
  spin<<<1, 1>>>(din, dack, dg, n);
  static long long h1[201], h2[201];
  for (unsigned k = 1; k <= n; k++) {
    long long t0 = now_ns();
    while (now_ns() - t0 < 20000) {}            // 20 us apart
    h1[k] = now_ns();
    *(volatile unsigned*)in = k;
    while (*(volatile unsigned*)ack != k) {}
    h2[k] = now_ns();
  }
  cudaDeviceSynchronize();
  long long best = -1, bo = 0, bh = 0;
  double sum_rtt = 0;
  for (unsigned k = 10; k <= n; k++) {
    long long rtt = h2[k] - h1[k];
    sum_rtt += rtt;
    if (best < 0 || rtt < best) { best = rtt; bo = (long long)g[k] - (h1[k] + h2[k]) / 2; bh = h1[k]; }
  }
  printf("{\"offset_ns\": %lld, \"host_ns\": %lld, \"min_rtt_ns\": %lld, \"mean_rtt_ns\": %.0f, \"samples\": %u, "
         "\"drift_ppm_within\": %.2f}\n", bo, bh, best, sum_rtt / (n - 9), n - 9,
         1e6 * (double)(((long long)g[n] - (h1[n] + h2[n]) / 2) - ((long long)g[10] - (h1[10] + h2[10]) / 2)) /
             (double)(h1[n] - h1[10]));
  return 0;
}
