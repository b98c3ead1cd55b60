// predict.cu -- application cycles from the representatives:
//   w_s = W_s / I,  IPC_s = x_rep / y_rep,  IPC = 1 / sum_s w_s / IPC_s,
//   C_pred = I / IPC = sum_s W_s * y_rep / x_rep                                        (A22)
// One block; each term in fp64 (W_s as a correctly rounded double of the u128), accumulated
// as a double-double (TwoSum) per thread and combined in a fixed tree, so the result is
// deterministic and within a few ulp of the exact rational value (tolerance 1e-9).
#include "kernels.cuh"

#define PR_THREADS 256

struct DD { double hi, lo; };

__device__ __forceinline__ DD dd_add(DD a, DD b) {
  double s = __dadd_rn(a.hi, b.hi);
  double bb = __dsub_rn(s, a.hi);
  double err = __dadd_rn(__dsub_rn(a.hi, __dsub_rn(s, bb)), __dsub_rn(b.hi, bb));
  double lo = __dadd_rn(__dadd_rn(a.lo, b.lo), err);
  double hi = __dadd_rn(s, lo);
  lo = __dsub_rn(lo, __dsub_rn(hi, s));
  DD r; r.hi = hi; r.lo = lo; return r;
}

__device__ __forceinline__ double u128_to_double(u64 lo, u64 hi) {
  // correctly rounded: keep the top 64 bits with a sticky bit, then scale exactly
  if (hi == 0) return __ull2double_rn(lo);
  int lz = __clzll(hi);
  int sh = 64 - lz;                       // bits of the value above the low 64, in [1, 64]
  u64 top, sticky;
  if (sh == 64) { top = hi; sticky = lo != 0; }
  else { top = (hi << lz) | (lo >> sh); sticky = (lo << lz) != 0; }
  return scalbn(__ull2double_rn(top | sticky), sh);  // >= 11 dropped bits: sticky LSB is exact
}

__global__ void __launch_bounds__(PR_THREADS)
k_predict(const u64* W, const u64* rx, const u64* ry, u32 nstrata, double* out) {
  pdl_begin();
  __shared__ DD s_c[PR_THREADS], s_i[PR_THREADS];
  __shared__ DD s_y[PR_THREADS];
  // block m predicts for the m-th cycle vector (one architecture each)
  ry += (u64)blockIdx.x * nstrata;
  out += 4 * (u64)blockIdx.x;
  DD c = {0.0, 0.0}, I = {0.0, 0.0}, Y = {0.0, 0.0};
  for (u32 s = threadIdx.x; s < nstrata; s += PR_THREADS) {
    double w = u128_to_double(W[2 * (u64)s], W[2 * (u64)s + 1]);
    double term = __ddiv_rn(__dmul_rn(w, __ull2double_rn(ry[s])), __ull2double_rn(rx[s]));
    DD t = {term, 0.0};
    c = dd_add(c, t);
    DD wi = {w, 0.0};
    I = dd_add(I, wi);
    DD yy = {__ull2double_rn(ry[s]), 0.0};
    Y = dd_add(Y, yy);
  }
  s_c[threadIdx.x] = c; s_i[threadIdx.x] = I; s_y[threadIdx.x] = Y;
  __syncthreads();
  for (int o = PR_THREADS / 2; o > 0; o >>= 1) {
    if ((int)threadIdx.x < o) {
      s_c[threadIdx.x] = dd_add(s_c[threadIdx.x], s_c[threadIdx.x + o]);
      s_i[threadIdx.x] = dd_add(s_i[threadIdx.x], s_i[threadIdx.x + o]);
      s_y[threadIdx.x] = dd_add(s_y[threadIdx.x], s_y[threadIdx.x + o]);
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    double cp = __dadd_rn(s_c[0].hi, s_c[0].lo);
    double ii = __dadd_rn(s_i[0].hi, s_i[0].lo);
    out[0] = cp;
    out[1] = __dadd_rn(s_y[0].hi, s_y[0].lo);
    out[2] = ii;
    out[3] = __ddiv_rn(ii, cp);
  }
}

// ry: [M][nstrata]; out: [M][4]
void launch_predict(const u64* W, const u64* rx, const u64* ry, u32 nstrata, u32 M, double* out,
                    cudaStream_t s) {
  if (M) SV_LAUNCH(k_predict, M, PR_THREADS, 0, s)(W, rx, ry, nstrata, out);
}
