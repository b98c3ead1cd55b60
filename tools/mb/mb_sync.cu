// Host wake-up latency after a kernel: cudaStreamSynchronize vs polling a flag the kernel writes
// to mapped pinned memory (after __threadfence_system).  nvcc -O2 -arch=sm_100a mb_sync.cu
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k_spin(unsigned long long ns, volatile unsigned long long* flag, unsigned long long seq) {
  unsigned long long t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 >= ns) break;
  }
  __threadfence_system();
  if (flag) *flag = seq;
}
int main() {
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  unsigned long long* h;
  cudaHostAlloc(&h, 64, cudaHostAllocMapped);
  unsigned long long* d;
  cudaHostGetDevicePointer((void**)&d, h, 0);
  using C = std::chrono::steady_clock;
  for (int mode = 0; mode < 2; mode++) {
    double tot = 0;
    const int N = 200;
    for (int i = 0; i < N + 10; i++) {
      *(volatile unsigned long long*)h = 0;
      auto t0 = C::now();
      k_spin<<<1, 1, 0, s>>>(200000, d, i + 1);   // 200 us of device time
      if (mode == 0) cudaStreamSynchronize(s);
      else while (*(volatile unsigned long long*)h != (unsigned long long)(i + 1)) {}
      auto t1 = C::now();
      if (i >= 10) tot += std::chrono::duration<double, std::micro>(t1 - t0).count() - 200.0;
      if (mode == 1) cudaStreamSynchronize(s);
    }
    printf("%s: launch + wake overhead %.1f us (kernel time subtracted)\n", mode ? "poll mapped flag" : "cudaStreamSynchronize", tot / N);
  }
  return 0;
}
