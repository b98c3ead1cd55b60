// Raw pinned host -> device bandwidth, one stream, 2 GB per copy (the e2e step's upload volume).
// nvcc -O2 -arch=sm_100a mb_h2d.cu
#include <cstdio>
#include <cuda_runtime.h>
int main() {
  const size_t B = 2000000000ull;
  void *h, *d;
  cudaHostAlloc(&h, B, cudaHostAllocDefault);
  cudaMalloc(&d, B);
  memset(h, 1, B);
  cudaStream_t s;
  cudaStreamCreate(&s);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int chunks : {1, 4, 16}) {
    for (int rep = 0; rep < 5; rep++) {
      cudaEventRecord(a, s);
      for (int c = 0; c < chunks; c++)
        cudaMemcpyAsync((char*)d + B / chunks * c, (char*)h + B / chunks * c, B / chunks, cudaMemcpyHostToDevice, s);
      cudaEventRecord(b, s);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      printf("chunks %2d: %.1f ms  %.1f GB/s\n", chunks, ms, B / ms / 1e6);
    }
  }
  return 0;
}
