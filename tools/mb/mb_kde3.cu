// Microbenchmark (not product code): FP64-pipe rate of the KDE term's dependency chain (no exp
// table) under variations of instruction form, terms in flight and warps per SM, to find what
// caps the 9-op chain at ~76% of the FP64 peak while independent DADD/DMUL streams reach 98%.
#include <cstdio>
typedef unsigned u32;
#define C_LOG2E_128 0x1.71547652b82fep+7
#define C_LN2_128 0x1.62e42fefa39efp-8
#define C_MAGIC 0x1.8p+52
#define C_TWO52 0x1.0p+52
#define C_P3 (-0x1.5555555555555p-3 * 0x1p-3)
__device__ double g_c[8] = {C_LOG2E_128, C_MAGIC, C_LN2_128, C_P3, 0.125, -0.5, 1.0, -C_MAGIC};
struct K { double L, M, LN, P3, P2, P1, P0, NM; };
// V: 0 full chain (9 FP64: dsub dmul dfma dadd dfma dfma dfma dfma dfma)
//    1 no kf (r from kb)                         8 ops
//    2 coefficients all in registers (no immediates)
//    3 r-fma with two operands (constant via immediate 0.5 instead of LN2 register)
//    4 final fma replaced by dadd (acc + p)      (2-operand)
//    5 chain of only DFMA(reg,reg,imm)           9 ops, all 2-reg
template <int V>
__device__ __forceinline__ double term(double gs, double xs, const K& k, double acc) {
  if (V == 5) {
    double a = __fma_rn(gs, xs, 0.5);
#pragma unroll
    for (int i = 0; i < 7; i++) a = __fma_rn(a, xs, 0.25);
    return __fma_rn(a, xs, acc);
  }
  double z = __dsub_rn(gs, xs);
  double u = __dmul_rn(z, z);
  double kb = __fma_rn(u, k.L, V == 2 ? k.M : C_MAGIC);
  double kf = V == 1 ? kb : (V == 2 ? __dadd_rn(kb, k.NM) : __dsub_rn(kb, C_MAGIC));
  double r = V == 3 ? __fma_rn(-kf, 0.5, u) : __fma_rn(-kf, k.LN, u);
  double p = V == 2 ? __fma_rn(k.P3, r, k.P2) : __fma_rn(k.P3, r, 0.125);
  p = V == 2 ? __fma_rn(p, r, k.P1) : __fma_rn(p, r, -0.5);
  p = V == 2 ? __fma_rn(p, r, k.P0) : __fma_rn(p, r, 1.0);
  if (V == 4) return __dadd_rn(acc, p);
  return __fma_rn(p, kf, acc);
}
template <int V, int U, int T>
__global__ void __launch_bounds__(T, 1) kern(double* out, int iters, double g0) {
  K k;
  asm volatile("mov.b64 %0, %1;" : "=d"(k.L) : "d"(g_c[0]));
  asm volatile("mov.b64 %0, %1;" : "=d"(k.M) : "d"(g_c[1]));
  asm volatile("mov.b64 %0, %1;" : "=d"(k.LN) : "d"(g_c[2]));
  asm volatile("mov.b64 %0, %1;" : "=d"(k.P3) : "d"(g_c[3]));
  asm volatile("mov.b64 %0, %1;" : "=d"(k.P2) : "d"(g_c[4]));
  asm volatile("mov.b64 %0, %1;" : "=d"(k.P1) : "d"(g_c[5]));
  asm volatile("mov.b64 %0, %1;" : "=d"(k.P0) : "d"(g_c[6]));
  asm volatile("mov.b64 %0, %1;" : "=d"(k.NM) : "d"(g_c[7]));
  double ac[U];
#pragma unroll
  for (int q = 0; q < U; q++) ac[q] = C_TWO52;
  double gs = g0 + threadIdx.x * 0.03;
  for (int it = 0; it < iters; it++) {
    double xs = it * 1e-3;
#pragma unroll
    for (int q = 0; q < U; q++) ac[q] = term<V>(gs, xs + q * 0.01, k, ac[q]);
  }
  double s = 0;
#pragma unroll
  for (int q = 0; q < U; q++) s += ac[q];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int V, int U, int T>
void run(const char* name, double* d, int iters) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  kern<V, U, T><<<148, T>>>(d, 10, 1.0);
  cudaEventRecord(a);
  kern<V, U, T><<<148, T>>>(d, iters, 1.0);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  double ops = 148.0 * T * iters * U * (V == 1 ? 8 : 9);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double peak = 148.0 * 64 * clk * 1e3;
  printf("%-34s T=%4d U=%2d %8.3f ms  %.1f%% of FP64 peak\n", name, T, U, ms, 100 * ops / ms / 1e9 / (peak / 1e12));
}
int main() {
  double* d; cudaMalloc(&d, 148 * 1024 * 8);
  int it = 3000;
  run<0, 16, 512>("full chain", d, it);
  run<0, 8, 512>("full chain", d, it);
  run<0, 24, 512>("full chain", d, it);
  run<0, 16, 256>("full chain", d, it);
  run<0, 8, 1024>("full chain", d, it);
  run<0, 16, 1024>("full chain", d, it);
  run<0, 4, 1024>("full chain", d, it);
  run<1, 16, 512>("no kf (8 ops)", d, it);
  run<2, 16, 512>("all-register coefficients", d, it);
  run<3, 16, 512>("r-fma with immediate", d, it);
  run<4, 16, 512>("final dadd", d, it);
  run<5, 16, 512>("9 x dfma(reg,reg,imm)", d, it);
  run<5, 8, 1024>("9 x dfma(reg,reg,imm)", d, it);
  return 0;
}
