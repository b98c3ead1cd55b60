// refine.cu -- one round of the Tier-3 refinement after the KDE (readings A11-A13):
//   * valleys of the (rank-reduced) density D by the integer hysteresis rule, cut thresholds
//     T = ceil(g_m), deduplicated and kept in (lo, hi]; no valley -> range bisection;
//   * exact moments of every candidate part [T_{q-1}, T_q) from the u128 prefix sums of x and
//     x^2 over the sorted keys (two binary searches per part, O(1) sums).
#include "kernels.cuh"

__device__ __forceinline__ double grid_pt_r(u64 lo, u64 hi, u32 j, u32 G) {
  return __dadd_rn(__ull2double_rn(lo),
                   __ddiv_rn(__ull2double_rn((hi - lo) * (u64)j), __uint2double_rn(G - 1)));
}

// Valley scan of one segment per warp: the warp stages D in shared memory (coalesced), lane 0
// runs the two-state hysteresis machine (A11): delta = max(1, max_j D_j >> shift); in seek_max
// track the running maximum and switch when D_j + delta <= max; in seek_min track the first run
// of the minimum and emit its midpoint once D_j >= min + delta.  Edges are never valleys.
#define VAL_WARPS 4
__global__ void __launch_bounds__(32 * VAL_WARPS)
k_valleys(const SegDev* segs, u32 nseg, u32 G, u32 shift, const u64* D, u64* T, u32 tstride,
          u32* nt, u32* kind) {
  u32 w = threadIdx.x >> 5;
  u32 s = blockIdx.x * VAL_WARPS + w;
  if (s >= nseg) return;
  const u64* d = D + 2 * (u64)s * G;
  // max over the segment (warp reduction on u128 as (hi, lo))
  u128 mx = 0;
  for (u32 j = lane_id(); j < G; j += 32) {
    u128 v = ((u128)d[2 * j + 1] << 64) | d[2 * j];
    mx = v > mx ? v : mx;
  }
  for (int o = 16; o > 0; o >>= 1) {
    u64 lo = __shfl_down_sync(0xffffffffu, (u64)mx, o);
    u64 hi = __shfl_down_sync(0xffffffffu, (u64)(mx >> 64), o);
    u128 v = ((u128)hi << 64) | lo;
    mx = v > mx ? v : mx;
  }
  if (lane_id() != 0) return;
  SegDev g = segs[s];
  u128 delta = mx >> shift;
  if (delta < 1) delta = 1;
  u64* Ts = T + (u64)s * tstride;
  u32 n = 0;
  bool seek_min = false;
  u128 top = ((u128)d[1] << 64) | d[0], low = 0;
  u32 a = 0, b = 0;
  for (u32 j = 1; j < G; j++) {
    u128 v = ((u128)d[2 * j + 1] << 64) | d[2 * j];
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
        if (th > g.lo && th <= g.hi && (n == 0 || Ts[n - 1] != th)) Ts[n++] = th;
        seek_min = false;
        top = v;
      }
    }
  }
  u32 k = 1;
  if (n == 0) { Ts[0] = (g.lo + g.hi + 1) >> 1; n = 1; k = 2; }  // value-range bisection (A13)
  nt[s] = n;
  kind[s] = k;
}

void launch_valleys(const SegDev* segs, u32 nseg, u32 G, u32 shift, const u64* D, u64* T,
                    u32 tstride, u32* nt, u32* kind, cudaStream_t s) {
  if (nseg) SV_LAUNCH(k_valleys, div_up(nseg, VAL_WARPS), 32 * VAL_WARPS, 0, s)(segs, nseg, G, shift, D, T,
                                                                        tstride, nt, kind);
}

__device__ __forceinline__ u64 lb_u64(const u64* a, u64 b, u64 e, u64 v) {
  while (b < e) {
    u64 m = (b + e) >> 1;
    if (a[m] < v) b = m + 1; else e = m;
  }
  return b;
}

__global__ void k_part_stats(const SegDev* segs, u32 nseg, const u64* T, u32 tstride,
                             const u32* nt, const u32* part_off, u32 nparts, const u64* keys,
                             u64 nkeys, u32 bx, const u64* P1, const u64* P2, u64* lanes, u64* mm,
                             u64* ab) {
  u32 p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= nparts) return;
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
  u64 n = ib - ia;
  u128 s1 = 0, s2 = 0;
  if (n) {
    s1 = (((u128)P1[2 * ib + 1] << 64) | P1[2 * ib]) - (((u128)P1[2 * ia + 1] << 64) | P1[2 * ia]);
    s2 = (((u128)P2[2 * ib + 1] << 64) | P2[2 * ib]) - (((u128)P2[2 * ia + 1] << 64) | P2[2 * ia]);
  }
  u64* L = lanes + (u64)p * MOM_LANES;
  L[0] = n;
  limbs_from_u128((u64)s1, (u64)(s1 >> 64), L + 1);
  limbs_from_u128((u64)s2, (u64)(s2 >> 64), L + 5);
  u64 xmask = (bx >= 64) ? ~0ull : ((1ull << bx) - 1);
  mm[p] = n ? (keys[ia] & xmask) : ~0ull;            // min (reduced with MIN)
  mm[nparts + p] = n ? (keys[ib - 1] & xmask) : 0;   // max (reduced with MAX)
  ab[2 * (u64)p] = a;
  ab[2 * (u64)p + 1] = b;
}

void launch_part_stats(const SegDev* segs, u32 nseg, const u64* T, u32 tstride, const u32* nt,
                       const u32* part_off, u32 nparts, const u64* keys, u64 nkeys, u32 bx,
                       const u64* P1, const u64* P2, u64* lanes, u64* mm, u64* ab, cudaStream_t s) {
  if (nparts)
    SV_LAUNCH(k_part_stats, div_up(nparts, 128), 128, 0, s)(segs, nseg, T, tstride, nt, part_off, nparts,
                                                      keys, nkeys, bx, P1, P2, lanes, mm, ab);
}
