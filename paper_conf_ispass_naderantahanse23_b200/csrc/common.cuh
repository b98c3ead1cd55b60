// common.cuh -- shared device/host helpers of libsieve (the product).  Nothing here is shared
// with oracle/ (the CPU oracle is a separate, independent implementation).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "sieve.h"

typedef unsigned long long u64;
typedef unsigned int u32;
typedef unsigned __int128 u128;

#define SIEVE_MAX_K 65536u
#define SIEVE_X_LIMIT (1ull << 44)

// ------------------------------------------------------------------------------------------
// error plumbing (host)
// ------------------------------------------------------------------------------------------
void sv_set_error(const std::string& msg);
int sv_fail(int code, const std::string& msg);
int sv_cuda(cudaError_t e, const char* what, int line);
#define SV_CUDA(x)                                         \
  do {                                                     \
    cudaError_t _e = (x);                                  \
    if (_e != cudaSuccess) return sv_cuda(_e, #x, __LINE__); \
  } while (0)
#define SV_TRY(x)            \
  do {                       \
    int _s = (x);            \
    if (_s != SIEVE_OK) return _s; \
  } while (0)

// ------------------------------------------------------------------------------------------
// reductions across ranks operate on u64 lanes; u128 values travel as 4 x 32-bit limbs
// ------------------------------------------------------------------------------------------
enum ReduceOp { RED_SUM = 0, RED_MIN = 1, RED_MAX = 2 };

__host__ __device__ inline void limbs_from_u128(u64 lo, u64 hi, u64* l) {
  l[0] = lo & 0xFFFFFFFFull;
  l[1] = lo >> 32;
  l[2] = hi & 0xFFFFFFFFull;
  l[3] = hi >> 32;
}

// normalise 4 lanes that each hold a sum of 32-bit limbs (< 2^64) back to a u128
__host__ __device__ inline void limbs_to_u128(const u64* l, u64* lo, u64* hi) {
  u64 c = 0;
  u64 w[4];
  for (int i = 0; i < 4; i++) {
    // l[i] + c can exceed 2^64 only if the true value overflowed u128 (never, by the bounds)
    u64 s = l[i] + c;
    w[i] = s & 0xFFFFFFFFull;
    c = (s >> 32) + ((s < l[i]) ? (1ull << 32) : 0ull);
  }
  *lo = w[0] | (w[1] << 32);
  *hi = w[2] | (w[3] << 32);
}

// device u128 accumulate into (lo, hi) words without __int128 on device paths
__device__ __forceinline__ void add128(u64& lo, u64& hi, u64 alo, u64 ahi) {
  u64 s = lo + alo;
  hi += ahi + (s < lo ? 1ull : 0ull);
  lo = s;
}

__device__ __forceinline__ u32 lane_id() { return threadIdx.x & 31u; }

// ------------------------------------------------------------------------------------------
// exact 256-bit arithmetic for the replicated decisions (host: tiers, parts; device: the part
// records' final / re-open flag), identical on both sides
// ------------------------------------------------------------------------------------------
struct W256 { u64 w[4]; };  // little-endian words

__host__ __device__ inline W256 w256_mul(u128 a, u128 b) {
  u64 A[2] = {(u64)a, (u64)(a >> 64)}, B[2] = {(u64)b, (u64)(b >> 64)};
  W256 r = {{0, 0, 0, 0}};
  for (int i = 0; i < 2; i++)
    for (int j = 0; j < 2; j++) {
      u128 p = (u128)A[i] * B[j];
      // add p at word i+j with carry propagation
      int k = i + j;
      u128 add = p;
      while (add && k < 4) {
        u128 s = (u128)r.w[k] + (u64)add;
        r.w[k] = (u64)s;
        add = (add >> 64) + (s >> 64);
        k++;
      }
    }
  return r;
}
__host__ __device__ inline W256 w256_mul_small(W256 a, u64 m) {
  W256 r;
  u128 c = 0;
  for (int i = 0; i < 4; i++) { u128 p = (u128)a.w[i] * m + c; r.w[i] = (u64)p; c = p >> 64; }
  return r;
}
__host__ __device__ inline W256 w256_sub(W256 a, W256 b) {
  W256 r;
  u64 br = 0;
  for (int i = 0; i < 4; i++) {
    u128 d = (u128)a.w[i] - b.w[i] - br;
    r.w[i] = (u64)d;
    br = (u64)(d >> 127);  // borrow if negative
  }
  return r;
}
__host__ __device__ inline bool w256_lt(W256 a, W256 b) {
  for (int i = 3; i >= 0; i--) if (a.w[i] != b.w[i]) return a.w[i] < b.w[i];
  return false;
}
// CoV < p/q  <=>  q^2 (n S2 - S1^2) < p^2 S1^2   (A1-A5)
__host__ __device__ inline bool cov_lt(u64 n, u128 s1, u128 s2, u32 p, u32 q) {
  W256 var_n2 = w256_sub(w256_mul(n, s2), w256_mul(s1, s1));
  return w256_lt(w256_mul_small(var_n2, (u64)q * q), w256_mul_small(w256_mul(s1, s1), (u64)p * p));
}


// ------------------------------------------------------------------------------------------
// launch helpers
// ------------------------------------------------------------------------------------------
static inline unsigned div_up(u64 a, u64 b) { return (unsigned)((a + b - 1) / b); }
int sv_num_sms();
// every kernel launch of the library goes through SV_LAUNCH so the process-wide launch
// count (sieve_kernel_launches) is exact
void sv_count_launch();

// Programmatic dependent launch (sm_90+): every kernel of the library is launched with
// programmatic stream serialisation and starts with pdl_begin(), which waits for the preceding
// grid to complete (its memory visible) before touching global memory, then lets the next
// kernel's blocks be scheduled as this grid's blocks retire.  The next kernel's launch and block
// dispatch overlap this one's tail instead of following it: the per-round chains of short
// kernels are launch-latency bound.
__device__ __forceinline__ void pdl_begin() {
  asm volatile("griddepcontrol.wait;\n\tgriddepcontrol.launch_dependents;" ::: "memory");
}
template <typename F>
struct PdlLaunch {
  F* k;
  dim3 g, b;
  size_t sm;
  cudaStream_t st;
  template <typename... A>
  void operator()(A... args) const {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = g;
    cfg.blockDim = b;
    cfg.dynamicSmemBytes = sm;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, k, args...);
  }
};
template <typename F>
inline PdlLaunch<F> sv_pdl(F* k, dim3 g, dim3 b, size_t sm, cudaStream_t st) { return PdlLaunch<F>{k, g, b, sm, st}; }
#define SV_LAUNCH(k, g, b, sm, st) sv_count_launch(), sv_pdl(k, dim3(g), dim3(b), (size_t)(sm), st)

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once per (kernel, device, size): launchers
// run on the host between synchronisations, where every driver call is GPU idle time
cudaError_t sv_set_smem(const void* fn, int bytes);
template <typename F>
inline cudaError_t sv_smem_attr(F* fn, int bytes) { return sv_set_smem((const void*)fn, bytes); }
