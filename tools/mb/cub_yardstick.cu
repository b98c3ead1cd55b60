// Yardstick (test/tool only, never on the product path): CUB's onesweep DeviceRadixSort on keys
// shaped like the round-1 cell sort of C4 -- 17.6M Tier-3 values, cell index = segment * 1024 +
// cell in the low 21 bits of a u64 key whose high bits carry x (the radix path's key layout) --
// against which the library's per-round cell grouping (bucket.cu) and its onesweep are compared.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o cub_yardstick cub_yardstick.cu
#include <cub/cub.cuh>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
typedef unsigned long long u64;

int main(int argc, char** argv) {
  const size_t n = argc > 1 ? strtoull(argv[1], 0, 10) : 17600000ull;
  const int ib = 21;
  std::mt19937_64 rng(0x51E7E004);
  std::vector<u64> h(n);
  // 2000 segments with Zipf-like sizes, values concentrated in a few cells per segment (modes)
  for (size_t i = 0; i < n; i++) {
    u64 r = rng();
    u64 seg = (u64)(2000.0 * std::pow((double)(r & 0xFFFFFF) / 16777216.0, 3.0));
    u64 mode = (r >> 24) % 6;
    u64 cell = (mode * 170 + ((r >> 32) % 40)) % 1024;
    u64 x = (r >> 20) & ((1ull << 40) - 1);
    h[i] = (x << ib) | (seg * 1024 + cell);
  }
  u64 *d_in, *d_out;
  cudaMalloc(&d_in, n * 8);
  cudaMalloc(&d_out, n * 8);
  cudaMemcpy(d_in, h.data(), n * 8, cudaMemcpyHostToDevice);
  size_t tb = 0;
  cub::DeviceRadixSort::SortKeys(nullptr, tb, d_in, d_out, (int)n, 0, ib);
  void* tmp;
  cudaMalloc(&tmp, tb);
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  for (int w = 0; w < 3; w++) cub::DeviceRadixSort::SortKeys(tmp, tb, d_in, d_out, (int)n, 0, ib);
  const int reps = 10;
  cudaEventRecord(a);
  for (int r = 0; r < reps; r++) cub::DeviceRadixSort::SortKeys(tmp, tb, d_in, d_out, (int)n, 0, ib);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  ms /= reps;
  const int passes = (ib + 7) / 8;
  printf("cub::DeviceRadixSort::SortKeys u64, bits [0,%d) (%d passes), n = %zu: %.4f ms  (%.0f GB/s at 16 B/key/pass)\n",
         ib, passes, n, ms, 16.0 * n * passes / (ms * 1e6));
  // the u32 cell index with a u64 payload (what a key-value sort of the same grouping moves)
  unsigned *k_in, *k_out;
  cudaMalloc(&k_in, n * 4); cudaMalloc(&k_out, n * 4);
  std::vector<unsigned> hk(n);
  for (size_t i = 0; i < n; i++) hk[i] = (unsigned)(h[i] & ((1u << ib) - 1));
  cudaMemcpy(k_in, hk.data(), n * 4, cudaMemcpyHostToDevice);
  size_t tb2 = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, tb2, k_in, k_out, d_in, d_out, (int)n, 0, ib);
  void* tmp2;
  cudaMalloc(&tmp2, tb2);
  for (int w = 0; w < 3; w++) cub::DeviceRadixSort::SortPairs(tmp2, tb2, k_in, k_out, d_in, d_out, (int)n, 0, ib);
  cudaEventRecord(a);
  for (int r = 0; r < reps; r++) cub::DeviceRadixSort::SortPairs(tmp2, tb2, k_in, k_out, d_in, d_out, (int)n, 0, ib);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  cudaEventElapsedTime(&ms, a, b);
  ms /= reps;
  printf("cub::DeviceRadixSort::SortPairs u32 key + u64 value, bits [0,%d), n = %zu: %.4f ms  (%.0f GB/s at 24 B/pair/pass)\n",
         ib, n, ms, 24.0 * n * passes / (ms * 1e6));
  return 0;
}
