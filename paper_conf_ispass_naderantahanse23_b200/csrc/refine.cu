// refine.cu -- one round of the Tier-3 refinement after the KDE (readings A11-A13):
//   * valleys of the (rank-reduced) density D by the integer hysteresis rule, cut thresholds
//     T = ceil(g_m), deduplicated and kept in (lo, hi]; no valley -> range bisection;
//   * exact moments of every candidate part [T_{q-1}, T_q) from the u128 prefix sums of x and
//     x^2 over the sorted keys (two binary searches per part, O(1) sums).
#include <algorithm>

#include "kernels.cuh"

__device__ __forceinline__ double grid_pt_r(u64 lo, u64 hi, u32 j, u32 G) {
  return __dadd_rn(__ull2double_rn(lo),
                   __ddiv_rn(__ull2double_rn((hi - lo) * (u64)j), __uint2double_rn(G - 1)));
}

// Valley scan of one segment per warp: the warp stages D in shared memory (coalesced) and
// reduces its maximum; then lane 0 runs the two-state hysteresis machine (A11) straight from
// shared memory (the loads do not depend on the state, so they run ahead of the dependent
// compare chain): delta = max(1, max_j D_j >> shift); in seek_max track the running maximum and
// switch when D_j + delta <= max; in seek_min track the first run of the minimum and emit its
// midpoint once D_j >= min + delta.  Edges are never valleys.
// the state machine over D (values read as (lo, hi) word pairs); V = u64 when every D_j < 2^63
// (then v + delta cannot wrap), else u128.  Returns the number of thresholds written to Ts.
template <typename V>
__device__ __forceinline__ u32 valley_machine(const u64* src, u32 G, V mx, u32 shift, const SegDev& g,
                                              u64* Ts) {
  V delta = shift >= 8 * sizeof(V) ? (V)0 : (V)(mx >> shift);
  if (delta < 1) delta = 1;
  u32 n = 0;
  bool seek_min = false;
  V top = sizeof(V) == 8 ? (V)src[0] : (V)(((u128)src[1] << 64) | src[0]), low = 0;
  u32 a = 0, b = 0;
  u64 last_th = 0;
#pragma unroll 4
  for (u32 j = 1; j < G; j++) {
    V v = sizeof(V) == 8 ? (V)src[2 * j] : (V)(((u128)src[2 * j + 1] << 64) | src[2 * j]);
    if (!seek_min) {
      if (v > top) top = v;
      if (v + delta <= top) { seek_min = true; low = v; a = b = j; }
    } else {
      if (v < low) { low = v; a = b = j; }
      else if (v == low && b == j - 1) { b = j; }
      else if (v >= low + delta) {
        u32 m = (a + b) >> 1;
        double gm = grid_pt_r(g.lo, g.hi, m, G);
        u64 th = (u64)ceil(gm);
        if (th > g.lo && th <= g.hi && (n == 0 || last_th != th)) {
          Ts[n] = th;
          last_th = th;
          n++;
        }
        seek_min = false;
        top = v;
      }
    }
  }
  return n;
}

#define VAL_WARPS 4
#define VAL_GMAX 2048   // segments with more grid points fall back to reading D from global memory
__global__ void __launch_bounds__(32 * VAL_WARPS)
k_valleys(const SegDev* segs, u32 nseg, u32 G, u32 shift, const u64* D, u64* T, u32 tstride,
          u32* nt, u32* kind) {
  extern __shared__ __align__(16) unsigned char vsm[];
  u32 w = threadIdx.x >> 5;
  u32 s = blockIdx.x * VAL_WARPS + w;
  if (s >= nseg) return;
  const u64* d = D + 2 * (u64)s * G;
  const bool staged = G <= VAL_GMAX;
  u64* sd = (u64*)vsm + (u64)w * 2 * G;
  // stage + max over the segment (warp reduction on u128 as (hi, lo))
  u128 mx = 0;
  for (u32 j = lane_id(); j < G; j += 32) {
    u64 lo = d[2 * j], hi = d[2 * j + 1];
    if (staged) { sd[2 * j] = lo; sd[2 * j + 1] = hi; }
    u128 v = ((u128)hi << 64) | lo;
    mx = v > mx ? v : mx;
  }
  for (int o = 16; o > 0; o >>= 1) {
    u64 lo = __shfl_down_sync(0xffffffffu, (u64)mx, o);
    u64 hi = __shfl_down_sync(0xffffffffu, (u64)(mx >> 64), o);
    u128 v = ((u128)hi << 64) | lo;
    mx = v > mx ? v : mx;
  }
  __syncwarp();
  if (lane_id() != 0) return;
  const u64* src = staged ? sd : d;
  SegDev g = segs[s];
  u64* Ts = T + (u64)s * tstride;
  u32 n = 0;
  if ((u64)(mx >> 63) == 0) n = valley_machine<u64>(src, G, (u64)mx, shift, g, Ts);  // usual: D < 2^63
  else n = valley_machine<u128>(src, G, mx, shift, g, Ts);
  u32 k = 1;
  if (n == 0) { Ts[0] = (g.lo + g.hi + 1) >> 1; n = 1; k = 2; }  // value-range bisection (A13)
  nt[s] = n;
  kind[s] = k;
}

void launch_valleys(const SegDev* segs, u32 nseg, u32 G, u32 shift, const u64* D, u64* T,
                    u32 tstride, u32* nt, u32* kind, cudaStream_t s) {
  if (!nseg) return;
  size_t smem = G <= VAL_GMAX ? (size_t)VAL_WARPS * 2 * G * 8 : 0;
  cudaFuncSetAttribute(k_valleys, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)((size_t)VAL_WARPS * 2 * VAL_GMAX * 8));
  SV_LAUNCH(k_valleys, div_up(nseg, VAL_WARPS), 32 * VAL_WARPS, smem, s)(segs, nseg, G, shift, D, T,
                                                                  tstride, nt, kind);
}

__device__ __forceinline__ u64 lb_u64(const u64* a, u64 b, u64 e, u64 v) {
  while (b < e) {
    u64 m = (b + e) >> 1;
    if (a[m] < v) b = m + 1; else e = m;
  }
  return b;
}

// One block per candidate part [a, b) of segment s (A13 f): its local index range [ia, ib) by
// two binary searches, then n = ib - ia and
//   S(ia, ib) = Pb[ib / B] - Pb[ia / B] + sum(keys[ib/B*B .. ib)) - sum(keys[ia/B*B .. ia))
// from the block-boundary prefixes Pb and at most two partial blocks (B = PREFIX_BLOCK), in
// exact modular u128 arithmetic.  Output: limb lanes (n, S1, S2), min / max, the interval.
#define PS_THREADS 256
__device__ __forceinline__ void ps_add(u64& s1, u64& s2lo, u64& s2hi, u64 x, bool neg) {
  u64 qlo = x * x, qhi = __umul64hi(x, x);
  if (neg) {  // two's complement of (x, x^2) in u64 / u128
    s1 -= x;
    u64 d = s2lo - qlo;
    s2hi -= qhi + (s2lo < qlo ? 1ull : 0ull);
    s2lo = d;
  } else {
    s1 += x;
    u64 t = s2lo + qlo;
    s2hi += qhi + (t < s2lo ? 1ull : 0ull);
    s2lo = t;
  }
}

__global__ void __launch_bounds__(PS_THREADS)
k_part_stats(const SegDev* segs, u32 nseg, const u64* T, u32 tstride, const u32* nt,
             const u32* part_off, const u32* d_nparts, u32 nparts_host, u32 mm_stride,
             const u64* keys, u64 nkeys, u32 bx, const u64* Pb, u64* lanes, u64* mm, u64* ab) {
  // the part count is either known on the host or read on the device (the part offsets were
  // scanned on the device: no host round trip between the valleys and the part moments)
  const u32 nparts = d_nparts ? *d_nparts : nparts_host;
  __shared__ u64 sh[4];
  __shared__ u64 r1[PS_THREADS / 32], r2l[PS_THREADS / 32], r2h[PS_THREADS / 32];
  const u64 xmask = (bx >= 64) ? ~0ull : ((1ull << bx) - 1);
  for (u32 p = blockIdx.x; p < nparts; p += gridDim.x) {
    if (threadIdx.x == 0) {
      u32 lo = 0, hi = nseg - 1;  // last segment with part_off[s] <= p
      while (lo < hi) {
        u32 m = (lo + hi + 1) >> 1;
        if (part_off[m] <= p) lo = m; else hi = m - 1;
      }
      u32 s = lo, q = p - part_off[s];
      SegDev g = segs[s];
      const u64* Ts = T + (u64)s * tstride;
      u64 a = q == 0 ? g.lo : Ts[q - 1];
      u64 b = q == nt[s] ? g.hi + 1 : Ts[q];
      u64 base = g.key_lo - g.lo;
      u64 ia = 0, ib = 0;
      if (nkeys) {
        ia = lb_u64(keys, g.begin, g.end, base + a);
        ib = lb_u64(keys, ia, g.end, base + b);
      }
      sh[0] = ia; sh[1] = ib;
      ab[4 * (u64)p] = a;        // value interval [a, b)
      ab[4 * (u64)p + 1] = b;
      ab[4 * (u64)p + 2] = ia;   // this rank's index range in the sorted keys (next round's
      ab[4 * (u64)p + 3] = ib;   // segment range if the part stays open)
    }
    __syncthreads();
    const u64 ia = sh[0], ib = sh[1];
    // this thread's share of the two partial blocks (x^2 < 2^88, so S2 needs a u128)
    u64 s1 = 0, s2lo = 0, s2hi = 0;
    if (ib > ia) {
      for (u64 j = (ib / PREFIX_BLOCK) * PREFIX_BLOCK + threadIdx.x; j < ib; j += PS_THREADS)
        ps_add(s1, s2lo, s2hi, keys[j] & xmask, false);
      for (u64 j = (ia / PREFIX_BLOCK) * PREFIX_BLOCK + threadIdx.x; j < ia; j += PS_THREADS)
        ps_add(s1, s2lo, s2hi, keys[j] & xmask, true);
    }
    // block reduction (modular; S1 partial fits u64 once combined with the prefix as u128 below)
    for (int o = 16; o > 0; o >>= 1) {
      u64 a1 = __shfl_down_sync(0xffffffffu, s1, o);
      u64 al = __shfl_down_sync(0xffffffffu, s2lo, o);
      u64 ah = __shfl_down_sync(0xffffffffu, s2hi, o);
      s1 += a1;
      u64 t = s2lo + al;
      s2hi += ah + (t < s2lo ? 1ull : 0ull);
      s2lo = t;
    }
    if (lane_id() == 0) { r1[threadIdx.x >> 5] = s1; r2l[threadIdx.x >> 5] = s2lo; r2h[threadIdx.x >> 5] = s2hi; }
    __syncthreads();
    if (threadIdx.x == 0) {
      u128 d1 = 0, d2 = 0;
      for (int w = 0; w < PS_THREADS / 32; w++) {
        d1 += (u128)(int64_t)r1[w];  // partial sums of S1 are < 2^57 in magnitude: sign-extend
        d2 += ((u128)r2h[w] << 64) | r2l[w];
      }
      u64 n = ib - ia;
      u128 S1 = 0, S2 = 0;
      if (n) {
        const u64* Pe = Pb + 4 * (ib / PREFIX_BLOCK);
        const u64* Pa = Pb + 4 * (ia / PREFIX_BLOCK);
        S1 = ((((u128)Pe[1] << 64) | Pe[0]) - (((u128)Pa[1] << 64) | Pa[0])) + d1;
        S2 = ((((u128)Pe[3] << 64) | Pe[2]) - (((u128)Pa[3] << 64) | Pa[2])) + d2;
      }
      u64* L = lanes + (u64)p * MOM_LANES;
      L[0] = n;
      limbs_from_u128((u64)S1, (u64)(S1 >> 64), L + 1);
      limbs_from_u128((u64)S2, (u64)(S2 >> 64), L + 5);
      mm[p] = n ? (keys[ia] & xmask) : ~0ull;                // min (reduced with MIN)
      mm[mm_stride + p] = n ? (keys[ib - 1] & xmask) : 0;   // max (reduced with MAX)
    }
  }
}

void launch_part_stats(const SegDev* segs, u32 nseg, const u64* T, u32 tstride, const u32* nt,
                       const u32* part_off, u32 nparts, const u64* keys, u64 nkeys, u32 bx,
                       const u64* Pb, u64* lanes, u64* mm, u64* ab, cudaStream_t s) {
  if (nparts)
    SV_LAUNCH(k_part_stats, nparts, PS_THREADS, 0, s)(segs, nseg, T, tstride, nt, part_off, nullptr,
                                                   nparts, nparts, keys, nkeys, bx, Pb, lanes, mm, ab);
}
