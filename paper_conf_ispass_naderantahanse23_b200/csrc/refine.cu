// refine.cu -- one round of the Tier-3 refinement after the KDE (readings A11-A13):
//   * valleys of the (rank-reduced) density D by the integer hysteresis rule, cut thresholds
//     T = ceil(g_m), deduplicated and kept in (lo, hi]; no valley -> range bisection;
//   (the exact moments of every candidate part [T_{q-1}, T_q) are in bucket.cu).
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

// The same machine run by a whole warp when every D_j < 2^63 (the usual case): each phase is a
// search for its switch point, 32 grid points at a time --
//   seek_max from p with running maximum top: the first j with D_j + delta <= max(top, D_p..D_j);
//   seek_min from s0 (low = D_s0): the first j with D_j >= min(D_s0..D_j) + delta; the valley's
//   run is the first index a of that minimum in [s0, j) and its contiguous run of equal values
//   [a, b] -- exactly the run the sequential machine tracks (a moves only on a strictly smaller
//   value, b extends only contiguously).
// Prefix maxima / minima by warp shuffles, switch points by ballots.  Identical output.
__device__ __forceinline__ u64 warp_prefix_max(u64 v) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    u64 t = __shfl_up_sync(0xffffffffu, v, o);
    if ((int)lane_id() >= o) v = t > v ? t : v;
  }
  return v;
}
__device__ __forceinline__ u64 warp_prefix_min(u64 v) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    u64 t = __shfl_up_sync(0xffffffffu, v, o);
    if ((int)lane_id() >= o) v = t < v ? t : v;
  }
  return v;
}
__device__ u32 valley_warp(const u64* src, u32 G, u64 mx, u32 shift, const SegDev& g, u64* Ts) {
  const u32 lane = lane_id();
  u64 delta = shift >= 64 ? 0 : (mx >> shift);
  if (delta < 1) delta = 1;
  auto val = [&](u32 j) -> u64 { return src[2 * j]; };  // low words (D < 2^63)
  u32 n = 0;
  u64 last_th = 0, top = val(0);
  u32 pos = 1;
  for (;;) {
    u32 s0 = G;  // seek_max -> seek_min switch
    for (u32 c = pos; c < G; c += 32) {
      const u32 j = c + lane;
      const u64 v = j < G ? val(j) : 0;
      u64 pm = warp_prefix_max(v);
      pm = pm > top ? pm : top;
      const u32 bal = __ballot_sync(0xffffffffu, j < G && v + delta <= pm);
      if (bal) { s0 = c + __ffs(bal) - 1; break; }
      top = __shfl_sync(0xffffffffu, pm, 31);
    }
    if (s0 >= G) break;
    u64 mn = val(s0);
    u32 e = G;  // seek_min -> seek_max switch
    for (u32 c = s0 + 1; c < G; c += 32) {
      const u32 j = c + lane;
      const u64 v = j < G ? val(j) : ~0ull;
      u64 pn = warp_prefix_min(v);
      pn = pn < mn ? pn : mn;
      const u32 bal = __ballot_sync(0xffffffffu, j < G && v >= pn + delta);
      if (bal) {
        e = c + __ffs(bal) - 1;
        mn = __shfl_sync(0xffffffffu, pn, __ffs(bal) - 1);  // = min over [s0, e)
        break;
      }
      mn = __shfl_sync(0xffffffffu, pn, 31);
    }
    if (e >= G) break;  // ends inside a trough: no valley (edges are never valleys)
    u32 a = s0, b;
    for (u32 c = s0; c < e; c += 32) {
      const u32 j = c + lane;
      const u32 bal = __ballot_sync(0xffffffffu, j < e && val(j) == mn);
      if (bal) { a = c + __ffs(bal) - 1; break; }
    }
    b = e - 1;
    for (u32 c = a + 1; c < e; c += 32) {
      const u32 j = c + lane;
      const u32 bal = __ballot_sync(0xffffffffu, j < e && val(j) != mn);
      if (bal) { b = c + __ffs(bal) - 2; break; }
    }
    const u32 m = (a + b) >> 1;
    const u64 th = (u64)ceil(grid_pt_r(g.lo, g.hi, m, G));
    if (th > g.lo && th <= g.hi && (n == 0 || last_th != th)) {
      if (lane == 0) Ts[n] = th;
      last_th = th;
      n++;
    }
    top = val(e);
    pos = e + 1;
  }
  return n;
}

#define VAL_WARPS 4
#define VAL_GMAX 2048   // segments with more grid points fall back to reading D from global memory
__global__ void __launch_bounds__(32 * VAL_WARPS)
k_valleys(const SegDev* segs, u32 nseg, u32 G, u32 shift, u64* D, u64* T, u32 tstride,
          u32* nt, u32* kind, bool writeback) {
  pdl_begin();
  extern __shared__ __align__(16) unsigned char vsm[];
  u32 w = threadIdx.x >> 5;
  u32 s = blockIdx.x * VAL_WARPS + w;
  if (s >= nseg) return;
  u64* d = D + 2 * (u64)s * G;
  const bool staged = G <= VAL_GMAX;
  u64* sd = (u64*)vsm + (u64)w * 2 * G;
  // The KDE leaves D_j as two u64 lanes (sum of the low 32-bit limbs, sum of the rest), summed
  // across ranks as they are: normalise to u128 here, stage, and reduce the maximum (warp
  // reduction on u128 as (hi, lo)).  The normalised D goes back to global memory when it is read
  // from there (large G) or read back (keep_debug).
  u128 mx = 0;
  for (u32 j = lane_id(); j < G; j += 32) {
    const u64 a = d[2 * j], b = d[2 * j + 1];
    const u64 lo = a + (b << 32);
    const u64 hi = (b >> 32) + (lo < a);
    if (staged) { sd[2 * j] = lo; sd[2 * j + 1] = hi; }
    if (writeback) { d[2 * j] = lo; d[2 * j + 1] = hi; }
    u128 v = ((u128)hi << 64) | lo;
    mx = v > mx ? v : mx;
  }
  for (int o = 16; o > 0; o >>= 1) {
    u64 lo = __shfl_xor_sync(0xffffffffu, (u64)mx, o);
    u64 hi = __shfl_xor_sync(0xffffffffu, (u64)(mx >> 64), o);
    u128 v = ((u128)hi << 64) | lo;
    mx = v > mx ? v : mx;
  }
  __syncwarp();
  const u64* src = staged ? sd : d;
  SegDev g = segs[s];
  u64* Ts = T + (u64)s * tstride;
  u32 n = 0;
  if ((u64)(mx >> 63) == 0) {
    n = valley_warp(src, G, (u64)mx, shift, g, Ts);  // usual: D < 2^63, the whole warp
    __syncwarp();
    if (lane_id() != 0) return;
  } else {
    if (lane_id() != 0) return;
    n = valley_machine<u128>(src, G, mx, shift, g, Ts);
  }
  u32 k = 1;
  if (n == 0) { Ts[0] = (g.lo + g.hi + 1) >> 1; n = 1; k = 2; }  // value-range bisection (A13)
  nt[s] = n;
  kind[s] = k;
}

void launch_valleys(const SegDev* segs, u32 nseg, u32 G, u32 shift, u64* D, u64* T,
                    u32 tstride, u32* nt, u32* kind, bool keep_D, cudaStream_t s) {
  if (!nseg) return;
  size_t smem = G <= VAL_GMAX ? (size_t)VAL_WARPS * 2 * G * 8 : 0;
  sv_smem_attr(k_valleys, (int)((size_t)VAL_WARPS * 2 * VAL_GMAX * 8));
  SV_LAUNCH(k_valleys, div_up(nseg, VAL_WARPS), 32 * VAL_WARPS, smem, s)(segs, nseg, G, shift, D, T,
                                                                  tstride, nt, kind, keep_D || G > VAL_GMAX);
}
