// microbenchmark: shared-memory atomic add throughput (u32 / u64 / f64), random addresses in a
// 2048-entry table, 1024 threads per block, one block per SM
#include <cstdio>
#include <cstdint>
template <typename T>
__global__ void k(T* out, int iters, unsigned seed) {
  __shared__ T tab[2048 * 2];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) tab[i] = 0;
  __syncthreads();
  unsigned s = seed ^ (threadIdx.x * 2654435761u) ^ (blockIdx.x * 40503u);
  for (int it = 0; it < iters; it++) {
    s = s * 1664525u + 1013904223u;
    unsigned a = (s >> 8) & 2047;
    atomicAdd(&tab[a], (T)(s & 255));
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = tab[5];
}
template <typename T>
float run(const char* name, int sms) {
  T* d; cudaMalloc(&d, sizeof(T) * sms);
  int iters = 1 << 14;
  k<T><<<sms, 1024>>>(d, 16, 1);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  k<T><<<sms, 1024>>>(d, iters, 7);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  double ops = (double)sms * 1024 * iters;
  printf("%s: %.3f ms, %.2f atomics/clk/SM (at 1.965 GHz)\n", name, ms, ops / (ms * 1e-3) / sms / 1.965e9);
  cudaFree(d);
  return ms;
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  run<unsigned>("u32", sms);
  run<unsigned long long>("u64", sms);
  run<double>("f64", sms);
  run<float>("f32", sms);
  return 0;
}
