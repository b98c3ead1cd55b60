// Microbenchmark (not product code): can the KDE term's "kf = kb - 1.5*2^52" (the integer k as
// a double, 1 of the 9 FP64-pipe ops) leave the FP64 pipe as an integer->double conversion of
// kb's low word?  Rate of the dependent chain with kf from DADD vs I2F.F64 (S32 / U32) vs
// F2F.F64.F32 of an I2F.F32, 14 terms in flight, 16 warps per SM (the kernel's shape).
#include <cstdio>
typedef unsigned u32;
#define C_LOG2E_128 0x1.71547652b82fep+7
#define C_LN2_128 0x1.62e42fefa39efp-8
#define C_MAGIC 0x1.8p+52
#define C_TWO52 0x1.0p+52
#define C_P3 (-0x1.5555555555555p-3 * 0x1p-3)
__device__ double g_c[3] = {C_LOG2E_128, C_MAGIC, C_LN2_128};
__constant__ double c_k[3] = {C_LOG2E_128, C_LN2_128, C_P3};
template <int V>
__device__ __forceinline__ double term(double gs, double xs, double L, double M, double acc) {
  double z = __dsub_rn(gs, xs);
  double u = __dmul_rn(z, z);
  double Lu = L;
  if (V == 4) asm volatile("ld.const.f64 %0, [c_k];" : "=d"(Lu));
  double kb = __fma_rn(u, Lu, M);
  double kf;
  if (V == 0) kf = __dsub_rn(kb, C_MAGIC);
  else if (V == 1) kf = __int2double_rn(__double2loint(kb));
  else if (V == 2) kf = __uint2double_rn((u32)__double2loint(kb));
  else if (V == 3) kf = (double)__int2float_rn(__double2loint(kb));
  else kf = __dsub_rn(kb, C_MAGIC);
  double c1 = c_k[1], c2 = c_k[2];
  if (V == 4) {   // constants through uniform registers: ld.const at the use, hoisted by ptxas
    asm volatile("ld.const.f64 %0, [c_k+8];" : "=d"(c1));
    asm volatile("ld.const.f64 %0, [c_k+16];" : "=d"(c2));
  }
  double r = __fma_rn(-kf, c1, u);
  double p = __fma_rn(c2, r, 0.125);
  p = __fma_rn(p, r, -0.5);
  p = __fma_rn(p, r, 1.0);
  return __fma_rn(p, z, acc);
}
template <int V, int U, int T>
__global__ void __launch_bounds__(T, 1) kern(double* out, int iters, double g0) {
  double L, M;
  asm volatile("mov.b64 %0, %1;" : "=d"(L) : "d"(g_c[0]));
  asm volatile("mov.b64 %0, %1;" : "=d"(M) : "d"(g_c[1]));
  double ac[U];
#pragma unroll
  for (int q = 0; q < U; q++) ac[q] = C_TWO52;
  double gs = g0 + threadIdx.x * 0.03;
  for (int it = 0; it < iters; it++) {
    double xs = it * 1e-3;
#pragma unroll
    for (int q = 0; q < U; q++) ac[q] = term<V>(gs, xs + q * 0.01, L, M, ac[q]);
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
  double terms = 148.0 * T * iters * U;
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double peak_terms = 148.0 * 64 * clk * 1e3 / 9;   // terms/s at 9 FP64 ops per term
  printf("%-28s T=%4d U=%2d %8.3f ms  %.1f%% of the 9-op term peak\n", name, T, U, ms,
         100 * terms / (ms * 1e-3) / peak_terms);
}
int main() {
  double* d; cudaMalloc(&d, 148 * 1024 * 8);
  int it = 3000;
  for (int rep = 0; rep < 2; rep++) {
    run<0, 14, 512>("kf = kb - magic (DADD)", d, it);
    run<1, 14, 512>("kf = I2F.F64.S32(lo(kb))", d, it);
    run<2, 14, 512>("kf = I2F.F64.U32(lo(kb))", d, it);
    run<3, 14, 512>("kf = F2F.F64(I2F.F32)", d, it);
    run<4, 14, 512>("constants in uniform regs", d, it);
    run<4, 16, 512>("constants in uniform regs", d, it);
    run<4, 12, 512>("constants in uniform regs", d, it);
  }
  return 0;
}
