// moments.cu -- pass A: one coalesced pass over (kernel id, instruction count, cycles) that
// reduces, per kernel, the exact moments n, S1 = sum x, S2 = sum x^2 and min / max x
// (CoV = sigma / mu with the population sigma; A1, A5), plus the totals C_meas = sum y
// and max x.
//
// B200 design: each block (one per SM, 1024 threads) keeps a privatised per-kernel table in
// shared memory.  sm_100a has no native 64-bit shared-memory add (it compiles to a CAS loop,
// measured 5x slower than 32-bit ATOMS), and 32-bit atomics with carry propagation serialise
// on their return values.  So x and x^2 are split into 15-bit limbs and each limb is added with
// a fire-and-forget 32-bit atomic into its own counter: no carries can occur before 2^17 - 1
// additions, so every 131071 rows the block flushes its limb counters (exactly, as u128) into
// its private 48-byte partial record per kernel in global memory and clears them.  Zero limbs
// are skipped (x < 2^30 needs 2 + 4 limb atomics plus the count).  min / max use a read-then-CAS
// that almost never takes the CAS.  A second kernel sums the blocks' partials exactly (u128) and
// emits 32-bit limbs in u64 lanes ready for a cross-rank all-reduce.
#include "kernels.cuh"

#define MOM_THREADS 1024
#ifndef MOM_PIPE
#define MOM_PIPE 1                            // next rows loaded while these are processed
#endif
#ifndef MOM_U
#define MOM_U 1                               // rows per thread per step (A/B pipelined: 1 < 2 < 4;
#endif                                        // unpipelined 2 was 10% slower than pipelined 1)
#define MOM_KT 2048                           // kernels per shared-memory pass (56 B each)
#define MOM_LB 15                             // limb bits
#define MOM_LMASK ((1u << MOM_LB) - 1u)
#define MOM_FLUSH ((1u << (32 - MOM_LB)) - 1u)  // rows between flushes: limb sums stay < 2^32
#define MOM_L1 3                              // limbs of x   (44 bits)
#define MOM_L2 6                              // limbs of x^2 (88 bits)
#define MOM_WORDS (1 + MOM_L1 + MOM_L2)       // count + limbs, u32 each

#ifndef MOM_MINB
#define MOM_MINB 1                            // resident blocks per SM (A/B on C4: 2 x 1024 threads caps the
                                              // kernel at 32 registers and spills: 0.72 -> 3.0 ms)
#endif

int moments_kt(u32 K) { return (int)(K < MOM_KT ? K : MOM_KT); }
// words between the two copies of the limb table: MOM_WORDS * kt rounded so that it is 16 mod 32
// (the copies' words for one kernel sit in opposite halves of the 32 banks)
__host__ __device__ inline u32 mom_copy_stride(u32 kt) {
  const u32 w = MOM_WORDS * kt;
  return w + ((16u - (w & 31u)) & 31u);
}
static size_t moments_smem(u32 kt, u32 nrep) { return (size_t)kt * 16 + (size_t)nrep * mom_copy_stride(kt) * 4; }
#ifndef MOM_REP
#define MOM_REP 2
#endif
#define MOM_SMEM_MAX (227 * 1024 - 2048)   // dynamic shared memory of one block (static part aside)
static u32 moments_nrep(u32 kt) { return MOM_REP >= 2 && moments_smem(kt, 2) <= MOM_SMEM_MAX ? 2u : 1u; }

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

__global__ void __launch_bounds__(MOM_THREADS, MOM_MINB)
k_moments(const u32* __restrict__ kid, const u64* __restrict__ x, const u64* __restrict__ y,
          u64 n, u32 K, u32 k0, u32 kt, u32 nrep, KMomPartial* __restrict__ part,
          u64* __restrict__ blk_tot, u64* errflags) {
  pdl_begin();
  extern __shared__ __align__(16) unsigned char smem[];
  u64* s_mn = (u64*)smem;                 // [kt]
  u64* s_mx = s_mn + kt;                  // [kt]
  u32* s_w = (u32*)(s_mx + kt);           // nrep x [MOM_WORDS][kt]: count, x limbs, x^2 limbs
  // nrep = 2: lanes 16..31 add into a second copy of the limb table, half a bank row away, so a
  // kernel that appears in both halves of a warp costs two parallel atomics, not two serial ones
  // (same-address collisions of Zipf-hot kernels dominated the shared-atomic wavefronts)
  const u32 cs = mom_copy_stride(kt);
  KMomPartial* rec = part + (u64)blockIdx.x * kt;
  for (u32 i = threadIdx.x; i < kt; i += blockDim.x) {
    s_mn[i] = ~0ull;
    s_mx[i] = 0;
    for (u32 r = 0; r < nrep; r++)
#pragma unroll
      for (int w = 0; w < MOM_WORDS; w++) s_w[r * cs + w * kt + i] = 0;
    KMomPartial z = {0, 0, 0, 0, 0, 0, 0};
    rec[i] = z;
  }
  __syncthreads();
  const bool totals = (k0 == 0);
  const bool use_y = totals && y;
  u64 chunk = (n + gridDim.x - 1) / gridDim.x;
  u64 b = (u64)blockIdx.x * chunk;
  u64 e = b + chunk < n ? b + chunk : n;
  u64 ylo = 0, yhi = 0, xmax = 0, err = 0;

  auto process = [&](u32 k, u64 v, u64 w) {
    if (totals) {
      if (k >= K) err |= ERRF_KID;
      if (v == 0 || v >= SIEVE_X_LIMIT) err |= ERRF_RANGE;
      xmax = v > xmax ? v : xmax;
      u64 s = ylo + w; yhi += s < ylo; ylo = s;
    }
    u32 l = k - k0;
    if (l >= kt || v == 0 || v >= SIEVE_X_LIMIT) return;
    u32* const sw = s_w + ((nrep == 2 && (lane_id() & 16u)) ? cs : 0u);
    atomicAdd(&sw[l], 1u);
#pragma unroll
    for (int i = 0; i < MOM_L1; i++) {
      u32 limb = (u32)(v >> (MOM_LB * i)) & MOM_LMASK;
      if (limb) atomicAdd(&sw[(1 + i) * kt + l], limb);
    }
    u64 sqlo = v * v, sqhi = __umul64hi(v, v);
#pragma unroll
    for (int i = 0; i < MOM_L2; i++) {
      int sh = MOM_LB * i;
      u64 bits = sh < 64 ? ((sqlo >> sh) | (sh ? (sqhi << (64 - sh)) : 0ull)) : (sqhi >> (sh - 64));
      u32 limb = (u32)bits & MOM_LMASK;
      if (limb) atomicAdd(&sw[(1 + MOM_L1 + i) * kt + l], limb);
    }
    atomic_min_u64_smem(&s_mn[l], v);
    atomic_max_u64_smem(&s_mx[l], v);
  };

  auto flush = [&]() {
    __syncthreads();
    for (u32 i = threadIdx.x; i < kt; i += blockDim.x) {
      u32 c = 0;
      for (u32 r = 0; r < nrep; r++) c += s_w[r * cs + i];
      if (!c) continue;
      u128 s1 = 0, s2 = 0;
      for (u32 r = 0; r < nrep; r++) {
        u32* sw = s_w + r * cs;
#pragma unroll
        for (int j = 0; j < MOM_L1; j++) {
          s1 += (u128)sw[(1 + j) * kt + i] << (MOM_LB * j);
          sw[(1 + j) * kt + i] = 0;
        }
#pragma unroll
        for (int j = 0; j < MOM_L2; j++) {
          s2 += (u128)sw[(1 + MOM_L1 + j) * kt + i] << (MOM_LB * j);
          sw[(1 + MOM_L1 + j) * kt + i] = 0;
        }
        sw[i] = 0;
      }
      KMomPartial r = rec[i];
      u128 a1 = (((u128)r.s1hi << 64) | r.s1lo) + s1;
      u128 a2 = (((u128)r.s2hi << 64) | r.s2lo) + s2;
      r.n += c;
      r.s1lo = (u64)a1; r.s1hi = (u32)(a1 >> 64);
      r.s2lo = (u64)a2; r.s2hi = (u64)(a2 >> 64);
      rec[i] = r;
    }
    __syncthreads();
  };

  const u64 step = blockDim.x;
  for (u64 c0 = b; c0 < e; c0 += MOM_FLUSH) {
    u64 c1 = c0 + MOM_FLUSH < e ? c0 + MOM_FLUSH : e;
    u64 i = c0 + threadIdx.x;
#if MOM_PIPE
    // the next MOM_U rows are loaded while these are processed
    u32 kk[MOM_U];
    u64 vv[MOM_U], ww[MOM_U];
    auto load = [&](u64 at, u32* k_, u64* v_, u64* w_) {
#pragma unroll
      for (int u = 0; u < MOM_U; u++) {
        const bool ok = at + u * step < c1;
        k_[u] = ok ? __ldcs(kid + at + u * step) : 0u;
        v_[u] = ok ? __ldcs(x + at + u * step) : 0ull;
        w_[u] = ok && use_y ? __ldcs(y + at + u * step) : 0ull;
      }
    };
    if (i + (MOM_U - 1) * step < c1) load(i, kk, vv, ww);
    for (; i + (MOM_U - 1) * step < c1; i += MOM_U * step) {
      u32 nk[MOM_U];
      u64 nv[MOM_U], nw[MOM_U];
      load(i + MOM_U * step, nk, nv, nw);   // rows past c1 load as 0 and are never processed
#pragma unroll
      for (int u = 0; u < MOM_U; u++) process(kk[u], vv[u], ww[u]);
#pragma unroll
      for (int u = 0; u < MOM_U; u++) { kk[u] = nk[u]; vv[u] = nv[u]; ww[u] = nw[u]; }
    }
#else
    for (; i + (MOM_U - 1) * step < c1; i += MOM_U * step) {
      u32 kk[MOM_U];
      u64 vv[MOM_U], ww[MOM_U];
#pragma unroll
      for (int u = 0; u < MOM_U; u++) {
        kk[u] = __ldcs(kid + i + u * step);
        vv[u] = __ldcs(x + i + u * step);
        ww[u] = use_y ? __ldcs(y + i + u * step) : 0ull;
      }
#pragma unroll
      for (int u = 0; u < MOM_U; u++) process(kk[u], vv[u], ww[u]);
    }
#endif
    for (; i < c1; i += step) process(__ldcs(kid + i), __ldcs(x + i), use_y ? __ldcs(y + i) : 0ull);
    flush();
  }
  for (u32 i = threadIdx.x; i < kt; i += blockDim.x) {
    rec[i].mn = s_mn[i];
    rec[i].mx = s_mx[i];
  }
  if (totals) {
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

// blocks of pass A: every SM holds as many blocks as its shared memory takes for this kt (two
// at K <= 2048: twice the warps to hide the shared-atomic latency), queried once per (device, kt)
int moments_grid(u32 kt) {
  static int cache[64][2] = {};
  int dev = 0;
  cudaGetDevice(&dev);
  int* e = cache[dev & 63];
  if (e[0] != (int)kt || e[1] < 1) {
    sv_smem_attr(k_moments, MOM_SMEM_MAX);
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_moments, MOM_THREADS, moments_smem(kt, moments_nrep(kt)));
    e[0] = (int)kt;
    e[1] = per_sm < 1 ? 1 : per_sm;
  }
  return sv_num_sms() * e[1];
}

void launch_moments(const u32* kid, const u64* x, const u64* y, u64 n, u32 K, u32 k0, u32 kt,
                    KMomPartial* part, u64* blk_tot, u64* errflags, int grid, cudaStream_t s) {
  sv_smem_attr(k_moments, MOM_SMEM_MAX);
  const u32 nrep = moments_nrep(kt);
  SV_LAUNCH(k_moments, grid, MOM_THREADS, moments_smem(kt, nrep), s)(kid, x, y, n, K, k0, kt, nrep, part, blk_tot,
                                                                     errflags);
}

// one warp per kernel: the lanes stride over the blocks' partials, exact u128 sums reduced by
// shuffles, emitted as limb lanes
__device__ __forceinline__ u128 shfl_xor_u128(u128 v, int o) {
  u64 lo = __shfl_xor_sync(0xffffffffu, (u64)v, o), hi = __shfl_xor_sync(0xffffffffu, (u64)(v >> 64), o);
  return ((u128)hi << 64) | lo;
}
__global__ void k_moments_reduce(const KMomPartial* __restrict__ part, int grid, u32 k0, u32 kt,
                                 u64* lanes, u64* mm, u64* local_n) {
  pdl_begin();
  u32 l = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (l >= kt) return;  // warp-uniform
  u128 n = 0, s1 = 0, s2 = 0;
  u64 mn = ~0ull, mx = 0;
  for (int b = lane_id(); b < grid; b += 32) {
    KMomPartial r = part[(u64)b * kt + l];
    n += r.n;
    s1 += ((u128)r.s1hi << 64) | r.s1lo;
    s2 += ((u128)r.s2hi << 64) | r.s2lo;
    mn = r.mn < mn ? r.mn : mn;
    mx = r.mx > mx ? r.mx : mx;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    n += shfl_xor_u128(n, o);
    s1 += shfl_xor_u128(s1, o);
    s2 += shfl_xor_u128(s2, o);
    u64 omn = __shfl_xor_sync(0xffffffffu, mn, o), omx = __shfl_xor_sync(0xffffffffu, mx, o);
    mn = omn < mn ? omn : mn;
    mx = omx > mx ? omx : mx;
  }
  if (lane_id() != 0) return;
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
  pdl_begin();
  if (blockIdx.x != 0 || threadIdx.x >= 32) return;
  u128 c = 0;
  u64 mx = 0;
  for (int b = lane_id(); b < grid; b += 32) {
    c += ((u128)blk_tot[3 * b + 1] << 64) | blk_tot[3 * b];
    mx = blk_tot[3 * b + 2] > mx ? blk_tot[3 * b + 2] : mx;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    c += shfl_xor_u128(c, o);
    u64 omx = __shfl_xor_sync(0xffffffffu, mx, o);
    mx = omx > mx ? omx : mx;
  }
  if (lane_id() != 0) return;
  limbs_from_u128((u64)c, (u64)(c >> 64), tot_lanes);
  tot_max[0] = mx;
}

void launch_moments_reduce(const KMomPartial* part, const u64* blk_tot, int grid, u32 k0, u32 kt,
                           u32 K, u64* lanes, u64* mm, u64* local_n, u64* tot_lanes, u64* tot_max,
                           bool do_totals, cudaStream_t s) {
  (void)K;
  SV_LAUNCH(k_moments_reduce, div_up((u64)kt * 32, 256), 256, 0, s)(part, grid, k0, kt, lanes, mm, local_n);
  if (do_totals) SV_LAUNCH(k_totals_reduce, 1, 32, 0, s)(blk_tot, grid, tot_lanes, tot_max);
}

// Tiers on the device (A1-A5), the host's exact test, so the round-1 grouping can be
// queued right behind pass A while the host takes the same decisions from its copy of the
// moments.  One block walks the kernels in order, 1024 at a time, carrying the Tier-3 rank and
// the running sum of the Tier-3 kernels' local rows.
__global__ void __launch_bounds__(1024) k_tiers(const u64* __restrict__ lanes, const u64* __restrict__ mm,
                                                const u64* __restrict__ local_n, u32 K, u32 p, u32 q,
                                                u32* __restrict__ t3rank, u32* __restrict__ seg_base,
                                                u32* __restrict__ t3kern, u32* __restrict__ counts) {
  pdl_begin();
  __shared__ u32 s_w[32], s_r[32];
  __shared__ u32 c_rank, c_rows;
  if (threadIdx.x == 0) { c_rank = 0; c_rows = 0; }
  __syncthreads();
  for (u32 k0 = 0; k0 < K; k0 += 1024) {
    const u32 k = k0 + threadIdx.x;
    bool t3 = false;
    u32 rows = 0;
    if (k < K) {
      const u64* L = lanes + (u64)k * MOM_LANES;
      if (L[0] && mm[2 * (u64)k] != mm[2 * (u64)k + 1]) {
        u64 a, b, c2, d;
        limbs_to_u128(L + 1, &a, &b);
        limbs_to_u128(L + 5, &c2, &d);
        t3 = !cov_lt(L[0], ((u128)b << 64) | a, ((u128)d << 64) | c2, p, q);
      }
      rows = t3 ? (u32)local_n[k] : 0u;
    }
    // block-wide exclusive scans of (is Tier-3, its rows)
    u32 f = t3 ? 1u : 0u, r = rows;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const u32 a = __shfl_up_sync(0xffffffffu, f, o), b = __shfl_up_sync(0xffffffffu, r, o);
      if ((int)lane_id() >= o) { f += a; r += b; }
    }
    const u32 w = threadIdx.x >> 5;
    if (lane_id() == 31) { s_w[w] = f; s_r[w] = r; }
    __syncthreads();
    if (w == 0) {
      u32 a = s_w[lane_id()], b = s_r[lane_id()];
      const u32 a0 = a, b0 = b;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const u32 x1 = __shfl_up_sync(0xffffffffu, a, o), x2 = __shfl_up_sync(0xffffffffu, b, o);
        if ((int)lane_id() >= o) { a += x1; b += x2; }
      }
      s_w[lane_id()] = a - a0;
      s_r[lane_id()] = b - b0;
    }
    __syncthreads();
    const u32 rank = c_rank + s_w[w] + f - (t3 ? 1u : 0u);
    const u32 base = c_rows + s_r[w] + r - rows;
    if (k < K) t3rank[k] = t3 ? rank : 0xFFFFFFFFu;
    if (t3) { seg_base[rank] = base; t3kern[rank] = k; }
    __syncthreads();
    if (threadIdx.x == 1023) { c_rank = rank + (t3 ? 1u : 0u); c_rows = base + rows; }
    __syncthreads();
  }
  if (threadIdx.x == 0) { counts[0] = c_rank; counts[1] = c_rows; }
}

void launch_tiers(const u64* lanes, const u64* mm, const u64* local_n, u32 K, u32 p, u32 q, u32* t3rank,
                  u32* seg_base, u32* t3kern, u32* counts, cudaStream_t s) {
  SV_LAUNCH(k_tiers, 1, 1024, 0, s)(lanes, mm, local_n, K, p, q, t3rank, seg_base, t3kern, counts);
}
