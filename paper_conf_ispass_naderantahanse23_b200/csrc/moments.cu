// moments.cu -- pass A: one coalesced pass over (kernel id, instruction count, cycles) that
// reduces, per kernel, the exact moments n, S1 = sum x, S2 = sum x^2 and min / max x
// (CoV = sigma / mu with the population sigma; A1, A5), plus the totals C_meas = sum y
// and max x.
//
// B200 design: each block keeps a privatised per-kernel table in shared memory.  B200 has no
// native 64-bit shared-memory add (it is a CAS loop, measured 5x slower than 32-bit ATOMS), so
// the wide sums are kept as 32-bit words updated by native 32-bit atomics with explicit carry
// propagation: atomicAdd returns the old word, the carry-out is added to the next word.  The
// final words are the exact sum of all added values regardless of interleaving.  min / max use
// a read-then-CAS that almost never takes the CAS after the first few invocations.  Blocks
// write one 48-byte partial per kernel; a second kernel sums the partials exactly (u128) and
// emits 32-bit limbs in u64 lanes ready for a cross-rank all-reduce.
#include "kernels.cuh"

#define MOM_THREADS 512
#define MOM_KT 2048  // kernels per shared-memory pass: 2048 * 44 B = 88 KB per block

int moments_kt(u32 K) { return (int)(K < MOM_KT ? K : MOM_KT); }
int moments_grid() { return 2 * sv_num_sms(); }

// add a value given as 32-bit words w[0..nw) into shared words a[0], a[stride], ...
template <int NW>
__device__ __forceinline__ void atomic_add_words(u32* a, u32 stride, const u32 (&w)[NW]) {
  u32 carry = 0;
#pragma unroll
  for (int i = 0; i < NW; i++) {
    u64 add = (u64)w[i] + carry;
    if (add == 0) { carry = 0; continue; }
    if (add == 0x100000000ull) { carry = 1; continue; }
    u32 old = atomicAdd(&a[i * stride], (u32)add);
    carry = ((u64)old + add) >> 32 ? 1u : 0u;
  }
}

__device__ __forceinline__ void atomic_min_u64_smem(u64* p, u64 v) {
  u64 cur = *(volatile u64*)p;
  while (v < cur) {
    u64 prev = atomicCAS((unsigned long long*)p, cur, v);
    if (prev == cur) break;
    cur = prev;
  }
}
__device__ __forceinline__ void atomic_max_u64_smem(u64* p, u64 v) {
  u64 cur = *(volatile u64*)p;
  while (v > cur) {
    u64 prev = atomicCAS((unsigned long long*)p, cur, v);
    if (prev == cur) break;
    cur = prev;
  }
}

__global__ void __launch_bounds__(MOM_THREADS)
k_moments(const u32* __restrict__ kid, const u64* __restrict__ x, const u64* __restrict__ y,
          u64 n, u32 K, u32 k0, u32 kt, KMomPartial* __restrict__ part,
          u64* __restrict__ blk_tot, u64* errflags) {
  extern __shared__ __align__(16) unsigned char smem[];
  u64* s_mn = (u64*)smem;                 // [kt]
  u64* s_mx = s_mn + kt;                  // [kt]
  u32* s_n = (u32*)(s_mx + kt);           // [kt]
  u32* s_s1 = s_n + kt;                   // [3][kt] words of S1
  u32* s_s2 = s_s1 + 3 * kt;              // [4][kt] words of S2
  for (u32 i = threadIdx.x; i < kt; i += blockDim.x) {
    s_mn[i] = ~0ull; s_mx[i] = 0; s_n[i] = 0;
    s_s1[i] = s_s1[kt + i] = s_s1[2 * kt + i] = 0;
    s_s2[i] = s_s2[kt + i] = s_s2[2 * kt + i] = s_s2[3 * kt + i] = 0;
  }
  __syncthreads();
  const bool totals = (k0 == 0);
  u64 chunk = (n + gridDim.x - 1) / gridDim.x;
  u64 b = (u64)blockIdx.x * chunk;
  u64 e = b + chunk < n ? b + chunk : n;
  u64 ylo = 0, yhi = 0, xmax = 0, err = 0;
  for (u64 i = b + threadIdx.x; i < e; i += blockDim.x) {
    u32 k = __ldcs(kid + i);
    u64 v = __ldcs(x + i);
    if (totals) {
      if (k >= K) err |= ERRF_KID;
      if (v == 0 || v >= SIEVE_X_LIMIT) err |= ERRF_RANGE;
      xmax = v > xmax ? v : xmax;
      if (y) { u64 w = __ldcs(y + i); u64 s = ylo + w; yhi += s < ylo; ylo = s; }
    }
    u32 l = k - k0;
    if (l >= kt || v == 0 || v >= SIEVE_X_LIMIT) continue;
    atomicAdd(&s_n[l], 1u);
    u32 w1[3] = {(u32)v, (u32)(v >> 32), 0u};
    atomic_add_words<3>(s_s1 + l, kt, w1);
    u64 sqlo = v * v, sqhi = __umul64hi(v, v);
    u32 w2[4] = {(u32)sqlo, (u32)(sqlo >> 32), (u32)sqhi, (u32)(sqhi >> 32)};
    atomic_add_words<4>(s_s2 + l, kt, w2);
    atomic_min_u64_smem(&s_mn[l], v);
    atomic_max_u64_smem(&s_mx[l], v);
  }
  __syncthreads();
  KMomPartial* out = part + (u64)blockIdx.x * kt;
  for (u32 i = threadIdx.x; i < kt; i += blockDim.x) {
    KMomPartial r;
    r.n = s_n[i];
    r.s1lo = (u64)s_s1[i] | ((u64)s_s1[kt + i] << 32);
    r.s1hi = s_s1[2 * kt + i];
    r.s2lo = (u64)s_s2[i] | ((u64)s_s2[kt + i] << 32);
    r.s2hi = (u64)s_s2[2 * kt + i] | ((u64)s_s2[3 * kt + i] << 32);
    r.mn = s_mn[i];
    r.mx = s_mx[i];
    out[i] = r;
  }
  if (totals) {
    // block reduction of (ylo, yhi), xmax, err through shared memory (reuse s_mn area after sync)
    __syncthreads();
    __shared__ u64 r_lo[MOM_THREADS / 32], r_hi[MOM_THREADS / 32], r_mx[MOM_THREADS / 32];
    for (int o = 16; o > 0; o >>= 1) {
      u64 olo = __shfl_down_sync(0xffffffffu, ylo, o);
      u64 ohi = __shfl_down_sync(0xffffffffu, yhi, o);
      u64 omx = __shfl_down_sync(0xffffffffu, xmax, o);
      u64 oer = __shfl_down_sync(0xffffffffu, err, o);
      u64 s = ylo + olo; yhi += ohi + (s < ylo); ylo = s;
      xmax = omx > xmax ? omx : xmax;
      err |= oer;
    }
    u32 w = threadIdx.x >> 5;
    if (lane_id() == 0) {
      r_lo[w] = ylo; r_hi[w] = yhi; r_mx[w] = xmax;
      // one 0/1 lane per error kind, so a cross-rank MAX reduction keeps each kind
      if (err & ERRF_KID) atomicMax((unsigned long long*)&errflags[0], 1ull);
      if (err & ERRF_RANGE) atomicMax((unsigned long long*)&errflags[1], 1ull);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      u64 lo = 0, hi = 0, mx = 0;
      for (u32 j = 0; j < blockDim.x / 32; j++) {
        u64 s = lo + r_lo[j]; hi += r_hi[j] + (s < lo); lo = s;
        mx = r_mx[j] > mx ? r_mx[j] : mx;
      }
      blk_tot[blockIdx.x * 3 + 0] = lo;
      blk_tot[blockIdx.x * 3 + 1] = hi;
      blk_tot[blockIdx.x * 3 + 2] = mx;
    }
  }
}

void launch_moments(const u32* kid, const u64* x, const u64* y, u64 n, u32 K, u32 k0, u32 kt,
                    KMomPartial* part, u64* blk_tot, u64* errflags, int grid, cudaStream_t s) {
  size_t smem = (size_t)kt * (8 + 8 + 4 + 12 + 16);
  cudaFuncSetAttribute(k_moments, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       MOM_KT * (8 + 8 + 4 + 12 + 16));
  SV_LAUNCH(k_moments, grid, MOM_THREADS, smem, s)(kid, x, y, n, K, k0, kt, part, blk_tot, errflags);
}

// one thread per kernel: exact u128 sum over the blocks' partials, emitted as limb lanes
__global__ void k_moments_reduce(const KMomPartial* __restrict__ part, int grid, u32 k0, u32 kt,
                                 u64* lanes, u64* mm, u64* local_n) {
  u32 l = blockIdx.x * blockDim.x + threadIdx.x;
  if (l >= kt) return;
  u128 n = 0, s1 = 0, s2 = 0;
  u64 mn = ~0ull, mx = 0;
  for (int b = 0; b < grid; b++) {
    KMomPartial r = part[(u64)b * kt + l];
    n += r.n;
    s1 += ((u128)r.s1hi << 64) | r.s1lo;
    s2 += ((u128)r.s2hi << 64) | r.s2lo;
    mn = r.mn < mn ? r.mn : mn;
    mx = r.mx > mx ? r.mx : mx;
  }
  u32 k = k0 + l;
  u64* L = lanes + (u64)k * MOM_LANES;
  L[0] = (u64)n;
  limbs_from_u128((u64)s1, (u64)(s1 >> 64), L + 1);
  limbs_from_u128((u64)s2, (u64)(s2 >> 64), L + 5);
  mm[2 * (u64)k] = mn;
  mm[2 * (u64)k + 1] = mx;
  local_n[k] = (u64)n;
}

__global__ void k_totals_reduce(const u64* blk_tot, int grid, u64* tot_lanes, u64* tot_max) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  u128 c = 0;
  u64 mx = 0;
  for (int b = 0; b < grid; b++) {
    c += ((u128)blk_tot[3 * b + 1] << 64) | blk_tot[3 * b];
    mx = blk_tot[3 * b + 2] > mx ? blk_tot[3 * b + 2] : mx;
  }
  limbs_from_u128((u64)c, (u64)(c >> 64), tot_lanes);
  tot_max[0] = mx;
}

void launch_moments_reduce(const KMomPartial* part, const u64* blk_tot, int grid, u32 k0, u32 kt,
                           u32 K, u64* lanes, u64* mm, u64* local_n, u64* tot_lanes, u64* tot_max,
                           bool do_totals, cudaStream_t s) {
  (void)K;
  SV_LAUNCH(k_moments_reduce, div_up(kt, 256), 256, 0, s)(part, grid, k0, kt, lanes, mm, local_n);
  if (do_totals) SV_LAUNCH(k_totals_reduce, 1, 32, 0, s)(blk_tot, grid, tot_lanes, tot_max);
}
