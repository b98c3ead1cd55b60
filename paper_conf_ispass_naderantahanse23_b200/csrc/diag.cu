// diag.cu -- within-stratum cycle variability (Fig. 4):
// per stratum the exact n, sum y and sum y^2 of its members' cycle counts, from one pass over
// (stratum id, cycles).  Same B200 design as pass A (moments.cu): a per-block table in shared
// memory with 15-bit limb counters updated by fire-and-forget 32-bit atomics, flushed exactly
// into a private per-block partial every 131071 rows, then an exact cross-block reduction into
// 32-bit-limb lanes ready for a cross-rank sum.  Cycles must be < 2^48 (4 limbs; y^2: 7 limbs).
#include "kernels.cuh"

#define GM_THREADS 1024
#define GM_KT 4608   // strata per shared-memory pass: 48 B each, 216 KB (C4's 3240 strata in one pass)
#define GM_LB 15
#define GM_LMASK ((1u << GM_LB) - 1u)
#define GM_FLUSH ((1u << (32 - GM_LB)) - 1u)
#define GM_L1 4   // limbs of y   (60 >= 48 bits)
#define GM_L2 7   // limbs of y^2 (105 >= 96 bits)
#define GM_WORDS (1 + GM_L1 + GM_L2)

int group_moments_kt(u32 ns) { return (int)(ns < GM_KT ? ns : GM_KT); }

__global__ void __launch_bounds__(GM_THREADS)
k_group_moments(const u32* __restrict__ sid, const u64* __restrict__ y, u64 n, u32 k0, u32 kt,
                GMomPartial* __restrict__ part, u64* errflag) {
  pdl_begin();
  extern __shared__ __align__(16) u32 s_w[];  // [GM_WORDS][kt]
  GMomPartial* rec = part + (u64)blockIdx.x * kt;
  for (u32 i = threadIdx.x; i < kt; i += blockDim.x) {
#pragma unroll
    for (int w = 0; w < GM_WORDS; w++) s_w[w * kt + i] = 0;
    GMomPartial z = {0, 0, 0, 0, 0};
    rec[i] = z;
  }
  __syncthreads();
  u64 chunk = (n + gridDim.x - 1) / gridDim.x;
  u64 b = (u64)blockIdx.x * chunk;
  u64 e = b + chunk < n ? b + chunk : n;
  bool bad = false;
  for (u64 c0 = b; c0 < e; c0 += GM_FLUSH) {
    u64 c1 = c0 + GM_FLUSH < e ? c0 + GM_FLUSH : e;
    // software pipelined: the next row's (stratum, cycles) load while this row is added
    u64 i = c0 + threadIdx.x;
    u32 nl = i < c1 ? __ldcs(sid + i) : 0u;
    u64 nv = i < c1 ? __ldcs(y + i) : 0ull;
    for (; i < c1; i += blockDim.x) {
      const u32 l = nl - k0;
      const u64 v = nv;
      const u64 i2 = i + blockDim.x;
      nl = i2 < c1 ? __ldcs(sid + i2) : 0u;
      nv = i2 < c1 ? __ldcs(y + i2) : 0ull;
      if (v >> 48) { bad = true; continue; }
      if (l >= kt) continue;
      atomicAdd(&s_w[l], 1u);
#pragma unroll
      for (int j = 0; j < GM_L1; j++) {
        u32 limb = (u32)(v >> (GM_LB * j)) & GM_LMASK;
        if (limb) atomicAdd(&s_w[(1 + j) * kt + l], limb);
      }
      u64 qlo = v * v, qhi = __umul64hi(v, v);
#pragma unroll
      for (int j = 0; j < GM_L2; j++) {
        int sh = GM_LB * j;
        u64 bits = sh < 64 ? ((qlo >> sh) | (sh ? (qhi << (64 - sh)) : 0ull)) : (qhi >> (sh - 64));
        u32 limb = (u32)bits & GM_LMASK;
        if (limb) atomicAdd(&s_w[(1 + GM_L1 + j) * kt + l], limb);
      }
    }
    __syncthreads();
    for (u32 i = threadIdx.x; i < kt; i += blockDim.x) {
      u32 c = s_w[i];
      if (!c) continue;
      u128 s1 = 0, s2 = 0;
#pragma unroll
      for (int j = 0; j < GM_L1; j++) { s1 += (u128)s_w[(1 + j) * kt + i] << (GM_LB * j); s_w[(1 + j) * kt + i] = 0; }
#pragma unroll
      for (int j = 0; j < GM_L2; j++) {
        s2 += (u128)s_w[(1 + GM_L1 + j) * kt + i] << (GM_LB * j);
        s_w[(1 + GM_L1 + j) * kt + i] = 0;
      }
      s_w[i] = 0;
      GMomPartial r = rec[i];
      u128 a1 = (((u128)r.s1hi << 64) | r.s1lo) + s1;
      u128 a2 = (((u128)r.s2hi << 64) | r.s2lo) + s2;
      r.n += c;
      r.s1lo = (u64)a1; r.s1hi = (u64)(a1 >> 64);
      r.s2lo = (u64)a2; r.s2hi = (u64)(a2 >> 64);
      rec[i] = r;
    }
    __syncthreads();
  }
  if (bad) atomicMax((unsigned long long*)errflag, 1ull);
}

// one thread per stratum: exact sum over the blocks' partials -> lanes n, S1 (4 limbs),
// S2 (6 limbs: a cross-rank S2 can exceed 2^128)
__global__ void k_group_moments_reduce(const GMomPartial* __restrict__ part, int grid, u32 k0,
                                       u32 kt, u64* lanes) {
  pdl_begin();
  u32 l = blockIdx.x * blockDim.x + threadIdx.x;
  if (l >= kt) return;
  u64 n = 0;
  u128 s1 = 0, s2 = 0;
  for (int b = 0; b < grid; b++) {
    GMomPartial r = part[(u64)b * kt + l];
    n += r.n;
    s1 += ((u128)r.s1hi << 64) | r.s1lo;
    s2 += ((u128)r.s2hi << 64) | r.s2lo;
  }
  u64* L = lanes + (u64)(k0 + l) * GM_LANES;
  L[0] = n;
  limbs_from_u128((u64)s1, (u64)(s1 >> 64), L + 1);
  limbs_from_u128((u64)s2, (u64)(s2 >> 64), L + 5);
  L[9] = 0;
  L[10] = 0;
}

void launch_group_moments(const u32* sid, const u64* y, u64 n, u32 nstrata, GMomPartial* part,
                          u64* lanes, u64* errflag, cudaStream_t s) {
  const u32 kt = (u32)group_moments_kt(nstrata);
  const int grid = sv_num_sms();
  size_t smem = (size_t)kt * GM_WORDS * 4;
  sv_smem_attr(k_group_moments, GM_KT * GM_WORDS * 4);
  for (u32 k0 = 0; k0 < nstrata; k0 += kt) {
    u32 kk = nstrata - k0 < kt ? nstrata - k0 : kt;
    if (n) SV_LAUNCH(k_group_moments, grid, GM_THREADS, smem, s)(sid, y, n, k0, kk, part, errflag);
    else cudaMemsetAsync(part, 0, (size_t)grid * kk * sizeof(GMomPartial), s);
    SV_LAUNCH(k_group_moments_reduce, div_up(kk, 256), 256, 0, s)(part, grid, k0, kk, lanes);
  }
}

size_t group_moments_part_bytes(u32 nstrata) {
  return (size_t)sv_num_sms() * group_moments_kt(nstrata) * sizeof(GMomPartial);
}
