// kde.cu -- fixed-point Gaussian KDE of every open Tier-3 segment on its G-point grid
// ("Kernel Density Estimation [8], [36]"; readings A6-A10 in DESIGN.md section 3):
//
//   g_j  = rn(lo) + rn((hi - lo) * j) / rn(G - 1)                      (A9)
//   z    = (g_j - rn(x)) * inv_h ;  t = (z * z) * 0.5
//   Q    = 0 if t > 37, else rint(det_exp(t) * 2^52)                  (A10)
//   D_j  = sum over the segment's values x of Q(x, g_j)   (exact integer sum, u128)
//
// det_exp(t) = ldexp(P(r), -k) with k = rint(t log2 e), r = t - k ln2 (two fma with a split ln2)
// and P the degree-13 Taylor polynomial of e^{-r} by Horner with fma.  Every floating-point
// step is an IEEE basic operation written with the _rn intrinsics (never contracted), so each
// term is bit-identical to the CPU oracle; the integer sum makes D independent of summation
// order, of the work decomposition and of the number of ranks.
//
// B200 mapping (the paper's scripts have no GPU design; this is new): the work is a gather over
// the SORTED values of each segment.  A work item is (segment, tile of KDE_TJ=128 grid points,
// chunk of <= KDE_CH=1024 values inside the tile's exact window |g - x| <= 8.7 h); a persistent
// grid pulls items from an atomic counter.  Each thread owns one grid point; the chunk's values
// are staged in shared memory as fp64 and read as warp broadcasts; each warp narrows the loop
// to its own window by binary search.  FP64 is on the CUDA cores (no contraction exists, so no
// tensor cores): ~24 FP64 pipe operations per in-window term.  Two bit tricks keep the
// conversions off the slow pipes: rint(t log2 e) = (t log2 e + 1.5 * 2^52) - 1.5 * 2^52 (its low
// word is k), and rint(P * 2^(52-k)) = bits(fma(P, 2^(52-k), 2^52)) - bits(2^52) because the
// product is exact and the sum lies in [2^52, 2^53] where the ulp is 1.
#include "kernels.cuh"

#define KDE_W 8.7  // window half-width in units of h: t > 37 is guaranteed beyond it

__device__ __forceinline__ double grid_pt(u64 lo, u64 hi, u32 j, u32 G) {
  return __dadd_rn(__ull2double_rn(lo),
                   __ddiv_rn(__ull2double_rn((hi - lo) * (u64)j), __uint2double_rn(G - 1)));
}

__device__ __forceinline__ u64 lower_bound_u64(const u64* a, u64 b, u64 e, u64 v) {
  while (b < e) {
    u64 m = (b + e) >> 1;
    if (a[m] < v) b = m + 1; else e = m;
  }
  return b;
}

// ------------------------------------------------------------------------------------------
__global__ void k_seg_ranges(SegDev* segs, u32 nseg, const u64* keys, u64 nkeys) {
  u32 s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= nseg) return;
  SegDev g = segs[s];
  u64 b = lower_bound_u64(keys, 0, nkeys, g.key_lo);
  u64 e = g.key_hi == ~0ull ? nkeys : lower_bound_u64(keys, b, nkeys, g.key_hi + 1);
  segs[s].begin = b;
  segs[s].end = e;
}

void launch_seg_ranges(SegDev* segs, u32 nseg, const u64* keys, u64 nkeys, cudaStream_t s) {
  if (nseg) SV_LAUNCH(k_seg_ranges, div_up(nseg, 128), 128, 0, s)(segs, nseg, keys, nkeys);
}

// per (segment, tile): the local index range of values inside the tile's window, and the
// number of KDE_CH-value chunks it takes
__global__ void k_kde_tiles(const SegDev* segs, u32 nseg, u32 G, u32 tps, const u64* keys,
                            u64* tile_range, u32* tile_items) {
  u64 id = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= (u64)nseg * tps) return;
  u32 s = (u32)(id / tps), t = (u32)(id % tps);
  SegDev g = segs[s];
  u32 j0 = t * KDE_TJ;
  u32 j1 = min(G - 1, j0 + KDE_TJ - 1);
  double w = __dmul_rn(KDE_W, g.h);
  double ga = __dsub_rn(grid_pt(g.lo, g.hi, j0, G), w);
  double gb = __dadd_rn(grid_pt(g.lo, g.hi, j1, G), w);
  u64 base = g.key_lo - g.lo;
  u64 xa = ga <= (double)g.lo ? g.lo : (u64)floor(ga);
  u64 xb = gb >= (double)g.hi ? g.hi : (u64)ceil(gb);
  u64 a = lower_bound_u64(keys, g.begin, g.end, base + xa);
  u64 z = lower_bound_u64(keys, a, g.end, base + xb + 1);
  tile_range[2 * id] = a;
  tile_range[2 * id + 1] = z;
  tile_items[id] = (u32)((z - a + KDE_CH - 1) / KDE_CH);
}

void scan_u32(const u32* in, u32* out, u64 n, void* temp, u32* total, cudaStream_t s);

int kde_plan(const SegDev* segs, u32 nseg, u32 G, const u64* keys, u64 nkeys, u64 xmask,
             u64* tile_range, u32* tile_items, void* scan_temp, u32* items_host, cudaStream_t s) {
  (void)nkeys; (void)xmask;
  u32 tps = div_up(G, KDE_TJ);
  u64 nt = (u64)nseg * tps;
  SV_LAUNCH(k_kde_tiles, div_up(nt, 128), 128, 0, s)(segs, nseg, G, tps, keys, tile_range, tile_items);
  // exclusive scan in place; tile_items[nt] receives the total
  scan_u32(tile_items, tile_items, nt, scan_temp, tile_items + nt, s);
  SV_CUDA(cudaMemcpyAsync(items_host, tile_items + nt, 4, cudaMemcpyDeviceToHost, s));
  SV_CUDA(cudaStreamSynchronize(s));
  return SIEVE_OK;
}

// ------------------------------------------------------------------------------------------
#define C_LOG2E 0x1.71547652b82fep+0
#define C_LN2_HI 0x1.62e42fee00000p-1
#define C_LN2_LO 0x1.a39ef35793c76p-33
#define C_MAGIC 0x1.8p+52   // 1.5 * 2^52
#define C_TWO52 0x1.0p+52

// Q(x, g) in fixed point 2^-52; returns 0 when t > 37
__device__ __forceinline__ u64 kde_term(double g, double xd, double inv_h, u32& inwin) {
  double z = __dmul_rn(__dsub_rn(g, xd), inv_h);
  double t = __dmul_rn(__dmul_rn(z, z), 0.5);
  if (t > 37.0) return 0;
  inwin++;
  double kb = __dadd_rn(__dmul_rn(t, C_LOG2E), C_MAGIC);
  double kf = __dsub_rn(kb, C_MAGIC);
  int k = __double2loint(kb);
  double r = __fma_rn(-kf, C_LN2_HI, t);
  r = __fma_rn(-kf, C_LN2_LO, r);
  double mr = -r;
  double p = 0x1.6124613a86d09p-33;                  // 1/13!
  p = __fma_rn(p, mr, 0x1.1eed8eff8d898p-29);        // 1/12!
  p = __fma_rn(p, mr, 0x1.ae64567f544e4p-26);        // 1/11!
  p = __fma_rn(p, mr, 0x1.27e4fb7789f5cp-22);        // 1/10!
  p = __fma_rn(p, mr, 0x1.71de3a556c734p-19);        // 1/9!
  p = __fma_rn(p, mr, 0x1.a01a01a01a01ap-16);        // 1/8!
  p = __fma_rn(p, mr, 0x1.a01a01a01a01ap-13);        // 1/7!
  p = __fma_rn(p, mr, 0x1.6c16c16c16c17p-10);        // 1/6!
  p = __fma_rn(p, mr, 0x1.1111111111111p-7);         // 1/5!
  p = __fma_rn(p, mr, 0x1.5555555555555p-5);         // 1/4!
  p = __fma_rn(p, mr, 0x1.5555555555555p-3);         // 1/3!
  p = __fma_rn(p, mr, 0x1.0p-1);                     // 1/2!
  p = __fma_rn(p, mr, 1.0);                          // 1/1!
  p = __fma_rn(p, mr, 1.0);                          // 1/0!
  double sc = __hiloint2double((1075 - k) << 20, 0); // 2^(52 - k), k in [0, 54)
  double q = __fma_rn(p, sc, C_TWO52);
  return (u64)__double_as_longlong(q) - 0x4330000000000000ull;
}

__global__ void __launch_bounds__(KDE_TJ)
k_kde(const SegDev* __restrict__ segs, u32 G, u32 tps, const u64* __restrict__ keys, u64 xmask,
      const u64* __restrict__ tile_range, const u32* __restrict__ tile_items, u32 ntiles,
      u32 items, u64* D, unsigned long long* counter, unsigned long long* terms) {
  __shared__ double sx[KDE_CH];
  __shared__ u32 s_item;
  u32 inwin = 0;
  for (;;) {
    if (threadIdx.x == 0) s_item = (u32)atomicAdd(counter, 1ull);
    __syncthreads();
    u32 item = s_item;
    if (item >= items) break;
    // tile containing the item: last tile with tile_items[tile] <= item
    u32 lo = 0, hi = ntiles - 1;
    while (lo < hi) {
      u32 m = (lo + hi + 1) >> 1;
      if (tile_items[m] <= item) lo = m; else hi = m - 1;
    }
    u32 tile = lo;
    u32 s = tile / tps, t = tile % tps;
    const SegDev& g = segs[s];
    u64 va = tile_range[2 * (u64)tile] + (u64)(item - tile_items[tile]) * KDE_CH;
    u64 ve = tile_range[2 * (u64)tile + 1];
    u32 len = (u32)min((u64)KDE_CH, ve - va);
    for (u32 i = threadIdx.x; i < len; i += KDE_TJ) sx[i] = __ull2double_rn(keys[va + i] & xmask);
    __syncthreads();
    u32 j = t * KDE_TJ + threadIdx.x;
    double inv_h = g.inv_h;
    double w = __dmul_rn(KDE_W, g.h);
    // this warp's window inside the chunk
    u32 jw0 = t * KDE_TJ + (threadIdx.x & ~31u);
    u32 jw1 = min(G - 1, jw0 + 31);
    u64 acc = 0;
    if (jw0 < G) {
      double wa = __dsub_rn(grid_pt(g.lo, g.hi, jw0, G), w);
      double wb = __dadd_rn(grid_pt(g.lo, g.hi, jw1, G), w);
      u32 a = 0, b = len;
      {  // first value >= wa
        u32 l = 0, r = len;
        while (l < r) { u32 m = (l + r) >> 1; if (sx[m] < wa) l = m + 1; else r = m; }
        a = l;
        l = a; r = len;
        while (l < r) { u32 m = (l + r) >> 1; if (sx[m] <= wb) l = m + 1; else r = m; }
        b = l;
      }
      double gj = grid_pt(g.lo, g.hi, j < G ? j : G - 1, G);
      u32 inwin0 = inwin;
#pragma unroll 2
      for (u32 i = a; i < b; i++) acc += kde_term(gj, sx[i], inv_h, inwin);
      if (j >= G) { acc = 0; inwin = inwin0; }
    }
    if (acc) {
      unsigned long long* d = (unsigned long long*)(D + 2 * ((u64)s * G + j));
      unsigned long long old = atomicAdd(d, (unsigned long long)acc);
      if (old + acc < old) atomicAdd(d + 1, 1ull);
    }
    __syncthreads();
  }
  if (terms) {
    for (int o = 16; o > 0; o >>= 1) inwin += __shfl_down_sync(0xffffffffu, inwin, o);
    if (lane_id() == 0 && inwin) atomicAdd(terms, (unsigned long long)inwin);
  }
}

void launch_kde(const SegDev* segs, u32 nseg, u32 G, const u64* keys, u64 xmask,
                const u64* tile_range, const u32* tile_items, u32 items, u64* D,
                unsigned long long* work_counter, unsigned long long* terms, cudaStream_t s) {
  if (items == 0) return;
  u32 tps = div_up(G, KDE_TJ);
  u32 ntiles = nseg * tps;
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_kde, KDE_TJ, 0);
  if (per_sm < 1) per_sm = 1;
  u32 grid = (u32)sv_num_sms() * (u32)per_sm;
  if (grid > items) grid = items;
  cudaMemsetAsync(work_counter, 0, 8, s);
  SV_LAUNCH(k_kde, grid, KDE_TJ, 0, s)(segs, G, tps, keys, xmask, tile_range, tile_items, ntiles, items, D,
                                 work_counter, terms);
}
