// bucket.cu -- the segmented sort of the Tier-3 values: once per refinement
// round, the values of the open segments are sorted by (open segment, grid cell).
//
// What the method needs from the order of the values (readings A9-A13): the KDE of a
// segment evaluates, for each tile of grid points, every value inside the tile's window
// |g - x| <= 7.6 h, and the part moments sum the values between two integer thresholds
// T = ceil(g_m).  Both only need the values GROUPED BY GRID CELL, not ordered inside a cell:
//   cell(x) = max { j : g_j <= x }        (g_0 = lo <= x <= hi, g_j the fp64 grid of A9)
// and, because x is an integer, x >= ceil(g_m) <=> x >= g_m <=> cell(x) >= m, so every part
// of a split is a contiguous run of cells (plus a filtered boundary cell when the no-valley
// bisection threshold falls inside a cell).  The KDE's densities are exact integer sums, so the
// order of values inside a cell cannot change any result.
//
// B200 mapping: sorting the full (kernel, x) keys took 7 onesweep digit passes (53-bit keys).
// Sorting by the cell index idx = segment * G + cell takes ceil(bitlen(#segments * G) / 8)
// passes (3 at C4), with x carried in the key's high bits: key = (x << ib) | idx.
//   k_grid_tab    : g_j of every open segment (L2-resident table, nseg x G doubles)
//   k_cellkey     : cell of every value (estimate + exact confirmation on the grid), its
//                   key, and the in-window KDE term count (diagnostic: grid points with
//                   rn(g - w) <= x <= rn(g + w), w = rn(sqrt(57) h)); values outside their
//                   segment's [lo, hi] get idx = #cells and sort to the end
//   radix_sort    : onesweep over bits [0, ib)
//   k_cell_offsets: off[c] = first position with idx >= c (c = 0..#cells)
// Hot cells (a narrow mode of a kernel whose range spans ten octaves falls into one cell) cost
// nothing extra: there is no per-cell atomic anywhere.  Round 1 reads the compacted Tier-3
// keys (segment = t3rank in the key's high bits); later rounds read, for each re-opened part,
// its superset range of whole cells in the previous round's sorted keys.
#include <algorithm>

#include "kernels.cuh"

#define BK_THREADS 256
#ifndef BK_U
#define BK_U 2            // values per thread in flight (A/B: 1, 2, 4 within noise; 8 slower)
#endif

__device__ __forceinline__ double grid_pt_b(u64 lo, u64 hi, u32 j, u32 G) {
  return __dadd_rn(__ull2double_rn(lo),
                   __ddiv_rn(__ull2double_rn((hi - lo) * (u64)j), __uint2double_rn(G - 1)));
}

__global__ void k_grid_tab(const SegDev* __restrict__ segs, u32 nseg, u32 G, double* __restrict__ gtab) {
  pdl_begin();
  u64 id = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= (u64)nseg * G) return;
  u32 s = (u32)(id / G), j = (u32)(id % G);
  gtab[id] = grid_pt_b(segs[s].lo, segs[s].hi, j, G);
}

void launch_grid_tab(const SegDev* segs, u32 nseg, u32 G, double* gtab, cudaStream_t s) {
  u64 n = (u64)nseg * G;
  if (n) SV_LAUNCH(k_grid_tab, div_up(n, 256), 256, 0, s)(segs, nseg, G, gtab);
}

// The per-value cell and in-window count evaluate the grid arithmetically (A9, one correctly
// rounded division each): a table lookup per grid point made the pass an L2-latency chain of
// random 8-byte gathers, the FP64 pipe has throughput to spare.
struct GridFn {
  double lod, Dm1;  // rn(lo), rn(G - 1)
  u64 D;            // hi - lo
  __device__ __forceinline__ double operator()(u32 j) const {
    return __dadd_rn(lod, __ddiv_rn(__ull2double_rn(D * (u64)j), Dm1));
  }
};

// max j with g_j <= x (lo <= x <= hi): the estimate from cq is exact unless x lies within
// rounding error of a grid point; a miss walks the grid (g is non-decreasing in j)
__device__ __forceinline__ u32 cell_arith(const GridFn& g, u32 G, double cq, u64 lo, u64 x) {
  double xd = __ull2double_rn(x);
  double e = __dmul_rn(__ull2double_rn(x - lo), cq);
  u32 j = e >= (double)(G - 1) ? G - 1 : (u32)e;
  if (g(j) <= xd && (j + 1 == G || g(j + 1) > xd)) return j;
  while (j + 1 < G && g(j + 1) <= xd) j++;
  while (j > 0 && g(j) > xd) j--;
  return j;
}

// number of grid points j with rn(g_j - w) <= x <= rn(g_j + w): the first j with
// rn(g_j + w) >= x and the last with rn(g_j - w) <= x, each estimated from cq and confirmed by
// its two neighbours; a miss walks the grid
__device__ __forceinline__ u32 inwin_count(const GridFn& g, u32 G, double cq, double w, u64 x) {
  const double xd = __ull2double_rn(x);
  const int Gi = (int)G;
  double ea = __dmul_rn(__dsub_rn(__dsub_rn(xd, w), g.lod), cq);
  double eb = __dmul_rn(__dsub_rn(__dadd_rn(xd, w), g.lod), cq);
  int a = ea <= 0.0 ? 0 : (ea >= (double)Gi ? Gi : (int)ceil(ea));
  int b = eb < 0.0 ? -1 : (eb >= (double)(Gi - 1) ? Gi - 1 : (int)floor(eb));
  bool oka = (a == Gi || __dadd_rn(g((u32)a), w) >= xd) && (a == 0 || __dadd_rn(g((u32)(a - 1)), w) < xd);
  if (!oka) {
    while (a > 0 && __dadd_rn(g((u32)(a - 1)), w) >= xd) a--;
    while (a < Gi && __dadd_rn(g((u32)a), w) < xd) a++;
  }
  bool okb = (b < 0 || __dsub_rn(g((u32)b), w) <= xd) && (b == Gi - 1 || __dsub_rn(g((u32)(b + 1)), w) > xd);
  if (!okb) {
    while (b + 1 < Gi && __dsub_rn(g((u32)(b + 1)), w) <= xd) b++;
    while (b >= 0 && __dsub_rn(g((u32)b), w) > xd) b--;
  }
  return b >= a ? (u32)(b - a + 1) : 0u;
}

// one thread per value (grid-stride): segment, cell, packed key, in-window term count; with
// chunks, nin = #chunks * BK_CHUNK and the padding of short chunks gets the sentinel key
__global__ void __launch_bounds__(BK_THREADS)
k_cellkey(const BucketChunk* __restrict__ chunks, u32 nchunks, const u64* __restrict__ in, u64 nin,
          u32 bx, u32 in_shift, const SegDev* __restrict__ segs, u32 G, const double* __restrict__ gtab,
          u32 ib, u32 ncell, u32 seg0, u64* __restrict__ out, unsigned long long* inwin,
          u32* __restrict__ ghist) {
  pdl_begin();
  // ghist != nullptr: the radix sort's digit histograms of the output keys over bits [0, ib)
  // (the cell index) are accumulated here, so the sort skips its own histogram read
  __shared__ u32 s_hist[3 * 256];
  const int npass = ghist ? (int)((ib + 7) / 8) : 0;   // ib <= 24 on this path (see launch)
  for (int i = threadIdx.x; i < npass * 256; i += BK_THREADS) s_hist[i] = 0;
  if (ghist) __syncthreads();
  const u32 nseg = ncell / G;
  const u64 xmask = bx >= 64 ? ~0ull : ((1ull << bx) - 1);
  u64 win = 0;
  // BK_U values per thread per step, all loaded before any is processed (latency hiding)
  const u64 stride = (u64)gridDim.x * BK_THREADS * BK_U;
  for (u64 i0 = (u64)blockIdx.x * BK_THREADS * BK_U + threadIdx.x; i0 < nin; i0 += stride) {
    u64 xs[BK_U];
    u32 ss[BK_U];
#pragma unroll
    for (int u = 0; u < BK_U; u++) {
      const u64 i = i0 + (u64)u * BK_THREADS;
      ss[u] = 0xFFFFFFFFu;  // sentinel: out of range / padding / another batch
      xs[u] = 0;
      if (i >= nin) continue;
      if (!chunks) {  // round 1: tagged Tier-3 keys, one output per input
        const u64 v = __ldcs(in + i);
        const u32 s = (u32)(v >> bx) - seg0;  // this batch's segments are t3rank seg0 .. seg0 + nseg - 1
        xs[u] = v & xmask;
        if (s < nseg) ss[u] = s;
      } else {        // later rounds: output i lies in chunk c (chunks hold BK_CHUNK values each)
        const BucketChunk ch = chunks[i / BK_CHUNK];
        const u32 r = (u32)(i % BK_CHUNK);
        if (r < ch.len) {  // else padding of a short chunk: sorts to the end
          ss[u] = ch.seg;
          xs[u] = __ldcs(in + ch.begin + r) >> in_shift;
        }
      }
    }
#pragma unroll
    for (int u = 0; u < BK_U; u++) {
    const u64 i = i0 + (u64)u * BK_THREADS;
    if (i >= nin) continue;
    const u64 x = xs[u];
    const u32 s = ss[u];
    if (s == 0xFFFFFFFFu) {
      out[i] = ncell;
      for (int p = 0; p < npass; p++) atomicAdd(&s_hist[p * 256 + ((ncell >> (8 * p)) & 255u)], 1u);
      continue;
    }
    const SegDev& g = segs[s];
    u64 lo = g.lo, hi = g.hi;
    u32 idx = ncell;
    if (x >= lo && x <= hi) {
      const GridFn gf{__ull2double_rn(lo), __uint2double_rn(G - 1), hi - lo};
      double cq = g.cq;
      idx = s * G + cell_arith(gf, G, cq, lo, x);
      if (inwin) win += inwin_count(gf, G, cq, __dmul_rn(KDE_WC, g.h), x);
    }
    out[i] = (x << ib) | idx;
    for (int p = 0; p < npass; p++) atomicAdd(&s_hist[p * 256 + ((idx >> (8 * p)) & 255u)], 1u);
    }
  }
  if (ghist) {
    __syncthreads();
    for (int i = threadIdx.x; i < npass * 256; i += BK_THREADS)
      if (s_hist[i]) atomicAdd(&ghist[i], s_hist[i]);
  }
  if (inwin) {
    for (int o = 16; o > 0; o >>= 1) win += __shfl_down_sync(0xffffffffu, win, o);
    if (lane_id() == 0 && win) atomicAdd(inwin, (unsigned long long)win);
  }
}

void launch_cellkey(const BucketChunk* chunks, const u64* in, u64 nin, u32 bx, u32 in_shift,
                    const SegDev* segs, u32 G, const double* gtab, u32 ib, u32 ncell, u32 seg0,
                    u64* out, unsigned long long* inwin, u32* ghist, cudaStream_t s) {
  if (!nin) return;
  if (ib > 24) ghist = nullptr;  // (the caller then lets the sort build its histograms)
  u64 grid = std::min<u64>((nin + BK_THREADS * BK_U - 1) / (BK_THREADS * BK_U), (u64)sv_num_sms() * 8);
  SV_LAUNCH(k_cellkey, (u32)grid, BK_THREADS, 0, s)(chunks, 0, in, nin, bx, in_shift, segs, G, gtab,
                                                    ib, ncell, seg0, out, inwin, ghist);
}

// off[c] = first position of the sorted keys with idx >= c, c = 0..ncell (position i writes the
// cells (idx(i-1), idx(i)]; position n writes the cells after the last key)
__global__ void k_cell_offsets(const u64* __restrict__ keys, u64 n, u32 ib, u32 ncell, u32* __restrict__ off) {
  pdl_begin();
  const u64 imask = (1ull << ib) - 1;
  const u64 stride = (u64)gridDim.x * blockDim.x;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i <= n; i += stride) {
    long long cur = i < n ? (long long)(__ldcs(keys + i) & imask) : (long long)ncell;
    long long prev = i ? (long long)(__ldcs(keys + i - 1) & imask) : -1;
    for (long long c = prev + 1; c <= cur; c++) off[c] = (u32)i;
  }
}

void launch_cell_offsets(const u64* keys, u64 n, u32 ib, u32 ncell, u32* off, cudaStream_t s) {
  u64 grid = std::min<u64>((n + 1 + 255) / 256, (u64)sv_num_sms() * 8);
  SV_LAUNCH(k_cell_offsets, (u32)grid, 256, 0, s)(keys, n, ib, ncell, off);
}

// ------------------------------------------------------------------------------------------
// Part moments (A13 f) over the bucketed values: part q of segment s is the value interval
// [a, b) (a = lo or T_{q-1}, b = T_q or hi + 1); its values lie in cells cell(a) .. cell(b - 1),
// i.e. in the contiguous range [off[cell(a)], off[cell(b - 1) + 1]), filtered to a <= x < b
// (only a bisection threshold can fall inside a cell).  The ranges are cut into work items of
// PS_CH values; a block reduces an item exactly (n, S1 u128, S2 u128, min, max) and adds it
// into the part's limb lanes with 64-bit atomics (sums of 32-bit limbs: exact, order-free).
// ------------------------------------------------------------------------------------------
#define PS_THREADS 256
#define PS_CH 8192      // values per work item

// part offsets on the device (one block): part_off[s] = sum over s' < s of (nt[s'] + 1),
// part_off[nseg] = number of parts -- the host needs no copy of the cut counts before the part
// moments are launched
__global__ void __launch_bounds__(1024) k_part_offsets(const u32* __restrict__ nt, u32 nseg, u32* part_off) {
  pdl_begin();
  __shared__ u32 carry;
  __shared__ u32 wsum[32];
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (u32 b = 0; b < nseg; b += 1024) {
    u32 s = b + threadIdx.x;
    u32 v = s < nseg ? nt[s] + 1 : 0;
    u32 inc = v;
    for (int o = 1; o < 32; o <<= 1) {
      u32 t = __shfl_up_sync(0xffffffffu, inc, o);
      if ((int)lane_id() >= o) inc += t;
    }
    if (lane_id() == 31) wsum[threadIdx.x >> 5] = inc;
    __syncthreads();
    if (threadIdx.x < 32) {
      u32 w = wsum[threadIdx.x], wi = w;
      for (int o = 1; o < 32; o <<= 1) {
        u32 t = __shfl_up_sync(0xffffffffu, wi, o);
        if ((int)lane_id() >= o) wi += t;
      }
      wsum[threadIdx.x] = wi - w;
    }
    __syncthreads();
    u32 c0 = carry;
    if (s < nseg) part_off[s] = c0 + wsum[threadIdx.x >> 5] + inc - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry = c0 + wsum[31] + inc;
    __syncthreads();
  }
  if (threadIdx.x == 0) part_off[nseg] = carry;
}

// one thread per part slot (p < cap; the live count is part_off[nseg]): value interval,
// bucketed range, work items (0 for dead slots)
__global__ void k_part_ranges(const SegDev* __restrict__ segs, u32 nseg, u32 G,
                              const double* __restrict__ gtab, const u32* __restrict__ off,
                              const u64* __restrict__ T, u32 tstride, const u32* __restrict__ nt,
                              const u32* __restrict__ part_off, u32 cap, u64* ab, u32* items) {
  pdl_begin();
  u32 p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= cap) return;
  if (p >= part_off[nseg]) { items[p] = 0; return; }
  u32 lo = 0, hi = nseg - 1;  // last segment with part_off[s] <= p
  while (lo < hi) {
    u32 m = (lo + hi + 1) >> 1;
    if (part_off[m] <= p) lo = m; else hi = m - 1;
  }
  u32 s = lo, q = p - part_off[s];
  const SegDev g = segs[s];
  const u64* Ts = T + (u64)s * tstride;
  u64 a = q == 0 ? g.lo : Ts[q - 1];
  u64 b = q == nt[s] ? g.hi + 1 : Ts[q];
  const double* gt = gtab + (u64)s * G;
  u32 ca = cell_of(gt, G, g.lo, g.cq, a), cb = cell_of(gt, G, g.lo, g.cq, b - 1);
  u64 ia = off[(u64)s * G + ca], ib = off[(u64)s * G + cb + 1];
  ab[4 * (u64)p] = a;        // value interval [a, b)
  ab[4 * (u64)p + 1] = b;
  ab[4 * (u64)p + 2] = ia;   // this rank's superset range in the bucketed values (the next
  ab[4 * (u64)p + 3] = ib;   // round's input if the part stays open)
  items[p] = (u32)((ib - ia + PS_CH - 1) / PS_CH);
}

// work items (part, chunk of PS_CH values of its range), pulled grid-stride; each block reduces
// its chunk exactly and adds it into the part's limb lanes / min / max with 64-bit atomics
__global__ void __launch_bounds__(PS_THREADS)
k_part_stats(const u64* __restrict__ ab, const u32* __restrict__ item_off, u32 cap,
             const u64* __restrict__ vals, u32 vshift, u64* lanes, u64* mm) {
  pdl_begin();
  __shared__ u64 r[PS_THREADS / 32][7];
  const u32 total = item_off[cap];
  for (u32 item = blockIdx.x; item < total; item += gridDim.x) {
    u32 lo = 0, hi = cap - 1;  // last part with item_off[p] <= item
    while (lo < hi) {
      u32 m = (lo + hi + 1) >> 1;
      if (item_off[m] <= item) lo = m; else hi = m - 1;
    }
    const u32 p = lo;
    const u64 a = ab[4 * (u64)p], b = ab[4 * (u64)p + 1];
    const u64 i0 = ab[4 * (u64)p + 2] + (u64)(item - item_off[p]) * PS_CH;
    const u64 i1 = min(i0 + PS_CH, ab[4 * (u64)p + 3]);
    u64 n = 0, s1lo = 0, s1hi = 0, s2lo = 0, s2hi = 0, mn = ~0ull, mx = 0;
    auto take = [&](u64 x) {
      x >>= vshift;
      if (x >= a && x < b) {
        n++;
        add128(s1lo, s1hi, x, 0);
        add128(s2lo, s2hi, x * x, __umul64hi(x, x));
        mn = x < mn ? x : mn;
        mx = x > mx ? x : mx;
      }
    };
    // eight values per thread loaded before they are added (one memory latency per eight)
    u64 i = i0 + threadIdx.x;
    for (; i + 7 * PS_THREADS < i1; i += 8 * PS_THREADS) {
      u64 v[8];
#pragma unroll
      for (int k = 0; k < 8; k++) v[k] = vals[i + (u64)k * PS_THREADS];
#pragma unroll
      for (int k = 0; k < 8; k++) take(v[k]);
    }
    for (; i < i1; i += PS_THREADS) take(vals[i]);
    for (int o = 16; o > 0; o >>= 1) {
      n += __shfl_down_sync(0xffffffffu, n, o);
      u64 al = __shfl_down_sync(0xffffffffu, s1lo, o), ah = __shfl_down_sync(0xffffffffu, s1hi, o);
      add128(s1lo, s1hi, al, ah);
      al = __shfl_down_sync(0xffffffffu, s2lo, o); ah = __shfl_down_sync(0xffffffffu, s2hi, o);
      add128(s2lo, s2hi, al, ah);
      u64 omn = __shfl_down_sync(0xffffffffu, mn, o), omx = __shfl_down_sync(0xffffffffu, mx, o);
      mn = omn < mn ? omn : mn;
      mx = omx > mx ? omx : mx;
    }
    const u32 w = threadIdx.x >> 5;
    if (lane_id() == 0) { r[w][0] = n; r[w][1] = s1lo; r[w][2] = s1hi; r[w][3] = s2lo; r[w][4] = s2hi; r[w][5] = mn; r[w][6] = mx; }
    __syncthreads();
    if (threadIdx.x == 0) {
      n = 0; s1lo = s1hi = s2lo = s2hi = 0; mn = ~0ull; mx = 0;
      for (int k = 0; k < PS_THREADS / 32; k++) {
        n += r[k][0];
        add128(s1lo, s1hi, r[k][1], r[k][2]);
        add128(s2lo, s2hi, r[k][3], r[k][4]);
        mn = r[k][5] < mn ? r[k][5] : mn;
        mx = r[k][6] > mx ? r[k][6] : mx;
      }
      if (n) {
        u64 l[8];
        limbs_from_u128(s1lo, s1hi, l);
        limbs_from_u128(s2lo, s2hi, l + 4);
        unsigned long long* L = (unsigned long long*)(lanes + (u64)p * MOM_LANES);
        atomicAdd(L, (unsigned long long)n);
        for (int k = 0; k < 8; k++)
          if (l[k]) atomicAdd(L + 1 + k, (unsigned long long)l[k]);
        atomicMin((unsigned long long*)&mm[p], (unsigned long long)mn);
        atomicMax((unsigned long long*)&mm[cap + p], (unsigned long long)mx);
      }
    }
    __syncthreads();
  }
}

void launch_part_offsets(const u32* nt, u32 nseg, u32* part_off, cudaStream_t s) {
  SV_LAUNCH(k_part_offsets, 1, 1024, 0, s)(nt, nseg, part_off);
}

void launch_part_stats(const SegDev* segs, u32 nseg, u32 G, const double* gtab, const u32* off,
                       const u64* T, u32 tstride, const u32* nt, const u32* part_off, u32 cap,
                       const u64* vals, u32 vshift, u32* items, void* scan_temp, u64* lanes, u64* mm,
                       u64* ab, cudaStream_t s) {
  if (!cap) return;
  SV_LAUNCH(k_part_ranges, div_up(cap, 128), 128, 0, s)(segs, nseg, G, gtab, off, T, tstride, nt,
                                                       part_off, cap, ab, items);
  scan_u32(items, items, cap, scan_temp, items + cap, s);
  SV_LAUNCH(k_part_stats, (u32)sv_num_sms() * 8, PS_THREADS, 0, s)(ab, items, cap, vals, vshift, lanes, mm);
}

// the round's results in one record per live part, written straight into mapped (zero-copy)
// host memory: out[0] = number of parts, then per part {lanes[9], min, max, ia, ib}
__device__ __forceinline__ void fill_part_record(u64* o, u32 p, u32 cap, const u64* __restrict__ lanes,
                                                      const u64* __restrict__ mm, const u64* __restrict__ ab,
                                                      u32 tp, u32 tq) {
  for (int k = 0; k < MOM_LANES; k++) o[k] = lanes[(u64)p * MOM_LANES + k];
  o[MOM_LANES] = mm[p];
  o[MOM_LANES + 1] = mm[cap + p];
  o[MOM_LANES + 2] = ab[4 * (u64)p + 2];
  o[MOM_LANES + 3] = ab[4 * (u64)p + 3];
  // the part's fate (A13 f): final stratum iff lo == hi or its exact CoV < theta = tp / tq (the
  // same u256 test as the tiering); the records are all-reduced already, so every rank agrees
  const u64* L = lanes + (u64)p * MOM_LANES;
  u64 s1lo, s1hi, s2lo, s2hi;
  limbs_to_u128(L + 1, &s1lo, &s1hi);
  limbs_to_u128(L + 5, &s2lo, &s2hi);
  const bool fin = L[0] != 0 && (mm[p] == mm[cap + p] ||
                                 cov_lt(L[0], ((u128)s1hi << 64) | s1lo, ((u128)s2hi << 64) | s2lo, tp, tq));
  o[MOM_LANES + 4] = fin ? 1ull : 0ull;
}

__global__ void k_part_pack(const u32* __restrict__ part_off, u32 nseg, u32 cap, const u64* __restrict__ lanes,
                            const u64* __restrict__ mm, const u64* __restrict__ ab, const u32* __restrict__ ntk,
                            u32 tp, u32 tq, u64* out) {
  pdl_begin();
  // the block's records are built in shared memory and written to the mapped host buffer as one
  // contiguous run of 8-byte words (consecutive threads, consecutive words: the PCIe writes
  // combine; a thread writing its own 112-byte record sent 8-byte writes 112 bytes apart)
  __shared__ u64 s_rec[128 * PART_REC];   // blockDim.x = 128
  const u32 nparts = part_off[nseg];
  const u32 p0 = blockIdx.x * blockDim.x;
  u32 p = p0 + threadIdx.x;
  if (p == 0) out[0] = nparts;
  // per segment: cut count and split kind (after the cap part slots)
  for (u32 q = p; q < nseg; q += gridDim.x * blockDim.x)
    out[1 + (u64)cap * PART_REC + q] = (u64)ntk[q] | ((u64)ntk[nseg + q] << 32);
  const u32 pend = min(nparts, cap);
  if (p0 >= pend) return;   // block-uniform
  if (p < pend) {
    u64* o = s_rec + threadIdx.x * PART_REC;
    fill_part_record(o, p, cap, lanes, mm, ab, tp, tq);
  }
  __syncthreads();
  const u32 nw = (min(pend, p0 + blockDim.x) - p0) * PART_REC;
  u64* dst = out + 1 + (u64)p0 * PART_REC;
  for (u32 w = threadIdx.x; w < nw; w += blockDim.x) dst[w] = s_rec[w];
}


void launch_part_pack(const u32* part_off, u32 nseg, u32 cap, const u64* lanes, const u64* mm,
                      const u64* ab, const u32* ntk, u32 tp, u32 tq, u64* out, cudaStream_t s) {
  SV_LAUNCH(k_part_pack, div_up(std::max<u32>(std::max(cap, nseg), 1), 128), 128, 0, s)(part_off, nseg, cap, lanes,
                                                                                    mm, ab, ntk, tp, tq, out);
}

// ==========================================================================================
// Cell GROUPING by counting sort (the default path for G <= GROUP_MAXG): the KDE windows and the
// part moments only need the values grouped by (segment, cell) -- the order inside a cell is
// irrelevant (exact integer sums, see the header) -- so no stable radix ranking is needed.
//   round 1   k_group_t3  : Tier-3 rows of the trace -> raw x grouped by segment (t3rank), at
//                           bases known from pass A's local counts; one shared atomic per Tier-3
//                           row and one global atomic per (tile, segment)
//   each round, over chunks of <= GR_CH values of one segment's range:
//             k_cell_hist : cell of every value (u16, 0xFFFF outside the segment's [lo, hi]) and
//                           the chunk's per-cell counts
//             k_cell_walk : per (segment, cell): offsets of the chunks inside the cell, cell total
//             scan_u32    : off[s * G + c] = first position of cell c of segment s (packed)
//             k_cell_scatter: values staged in shared memory in cell order, written out in runs
// Traffic per value and round: 8 B read (hist) + 2 B cell write + (8 + 2) B read + 8 B write
// (scatter), against 16 B per onesweep pass x 3 passes + 16 B for the radix path's cell keys.
// ==========================================================================================
#define GR_THREADS 512
#define GR_CH 8192          // values per chunk (one block), 16 per thread
#define GT_ROWS 16          // trace rows per thread per tile in k_group_t3
#define GT_SMEM_MAX GROUP_T3_SMEM_MAX   // segments handled with a shared-memory counter table

__global__ void __launch_bounds__(GR_THREADS)
k_group_t3(const u32* __restrict__ kid, const u64* __restrict__ x, u64 n, const u32* __restrict__ t3rank,
           u32 n_t3, const u32* __restrict__ seg_base, u32* __restrict__ cursor, u64* __restrict__ out) {
  pdl_begin();
  extern __shared__ u32 s_cnt[];      // [n_t3]: tile counts, then the tile's output bases
  __shared__ u32 s_list[GR_THREADS * GT_ROWS];
  __shared__ u32 s_nlist;
  const bool smem = n_t3 <= GT_SMEM_MAX;
  if (smem)
    for (u32 i = threadIdx.x; i < n_t3; i += GR_THREADS) s_cnt[i] = 0;
  if (threadIdx.x == 0) s_nlist = 0;
  __syncthreads();
  const u64 tile = (u64)GR_THREADS * GT_ROWS;
  for (u64 base = (u64)blockIdx.x * tile; base < n; base += (u64)gridDim.x * tile) {
    u32 t[GT_ROWS], r[GT_ROWS];
    u64 v[GT_ROWS];
#pragma unroll
    for (int j = 0; j < GT_ROWS; j++) {   // all loads first
      const u64 i = base + (u64)j * GR_THREADS + threadIdx.x;
      const bool ok = i < n;
      t[j] = ok ? __ldcs(kid + i) : 0u;
      v[j] = ok ? __ldcs(x + i) : 0ull;
      if (!ok) t[j] = 0xFFFFFFFFu;
    }
#pragma unroll
    for (int j = 0; j < GT_ROWS; j++) {
      if (t[j] != 0xFFFFFFFFu) t[j] = __ldg(t3rank + t[j]);
      if (t[j] == 0xFFFFFFFFu) continue;
      if (smem) {
        r[j] = atomicAdd(&s_cnt[t[j]], 1u);
        if (r[j] == 0) s_list[atomicAdd(&s_nlist, 1u)] = t[j];
      } else {
        r[j] = seg_base[t[j]] + atomicAdd(&cursor[t[j]], 1u);
      }
    }
    if (smem) {
      __syncthreads();
      const u32 nl = s_nlist;
      for (u32 q = threadIdx.x; q < nl; q += GR_THREADS) {  // reserve one range per segment
        const u32 s = s_list[q];
        s_cnt[s] = seg_base[s] + atomicAdd(&cursor[s], s_cnt[s]);
      }
      __syncthreads();
#pragma unroll
      for (int j = 0; j < GT_ROWS; j++)
        if (t[j] != 0xFFFFFFFFu) out[s_cnt[t[j]] + r[j]] = v[j];
      __syncthreads();
      for (u32 q = threadIdx.x; q < nl; q += GR_THREADS) s_cnt[s_list[q]] = 0;
      if (threadIdx.x == 0) s_nlist = 0;
      __syncthreads();
    } else {
#pragma unroll
      for (int j = 0; j < GT_ROWS; j++)
        if (t[j] != 0xFFFFFFFFu) out[r[j]] = v[j];
    }
  }
}

// The default round-1 grouping (n_t3 <= GT_SMEM_MAX): blocks own fixed contiguous row ranges;
// k_t3_count counts each block's Tier-3 rows per segment, k_t3_offsets turns the counts into
// each (segment, block) output base, and k_t3_scatter writes every Tier-3 row at its block's
// next position of its segment (a shared-memory atomic): no global atomics, no per-tile barriers.
#define T3_THREADS 512
#define T3_SC_THREADS 1024   // k_t3_scatter (one block per SM when it reuses pass A's row ranges)
#define T3_U 8               // rows per thread in flight
__device__ __forceinline__ void t3_range(u64 n, u32 nb, u32 b, u64* r0, u64* r1) {
  const u64 chunk = (n + nb - 1) / nb;
  *r0 = min(n, (u64)b * chunk);
  *r1 = min(n, *r0 + chunk);
}

__global__ void __launch_bounds__(T3_THREADS)
k_t3_count(const u32* __restrict__ kid, const u64* __restrict__ x, u64 n, u32 K, const u32* __restrict__ t3rank,
           u32 n_t3, const u32* __restrict__ n_t3_dev, u32* __restrict__ cnt) {
  pdl_begin();
  extern __shared__ u32 s_c[];   // [n_t3]
  if (n_t3_dev) n_t3 = *n_t3_dev;
  for (u32 i = threadIdx.x; i < n_t3; i += T3_THREADS) s_c[i] = 0;
  __syncthreads();
  u64 r0, r1;
  t3_range(n, gridDim.x, blockIdx.x, &r0, &r1);
  for (u64 i0 = r0 + threadIdx.x; i0 < r1; i0 += (u64)T3_THREADS * T3_U) {
    u32 k[T3_U];
#pragma unroll
    for (int u = 0; u < T3_U; u++) {
      const u64 i = i0 + (u64)u * T3_THREADS;
      k[u] = i < r1 ? __ldcs(kid + i) : 0xFFFFFFFFu;
    }
#pragma unroll
    for (int u = 0; u < T3_U; u++) {
      const u32 t = k[u] < K ? __ldg(t3rank + k[u]) : 0xFFFFFFFFu;
      if (t == 0xFFFFFFFFu) continue;
      const u64 v = __ldcs(x + i0 + (u64)u * T3_THREADS);
      if (v != 0 && v < SIEVE_X_LIMIT) atomicAdd(&s_c[t], 1u);   // the rows pass A counts
    }
  }
  __syncthreads();
  for (u32 t = threadIdx.x; t < n_t3; t += T3_THREADS) cnt[(u64)t * gridDim.x + blockIdx.x] = s_c[t];
}

// one warp per segment: exclusive scan of its per-block counts, offset by the segment's base;
// part != nullptr: the counts are pass A's per-block kernel counts (part[b * kt + kernel].n, the
// same row ranges), t3kern[t] = the kernel of segment t
__global__ void k_t3_offsets(u32* __restrict__ cnt, u32 nb, u32 n_t3, const u32* __restrict__ n_t3_dev,
                             const u32* __restrict__ seg_base, const KMomPartial* __restrict__ part, u32 kt,
                             const u32* __restrict__ t3kern) {
  pdl_begin();
  const u32 t = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (n_t3_dev) n_t3 = *n_t3_dev;
  if (t >= n_t3) return;
  u32 carry = seg_base[t];
  u32* row = cnt + (u64)t * nb;
  const u32 kk = part ? t3kern[t] : 0u;
  for (u32 b0 = 0; b0 < nb; b0 += 32) {
    const u32 b = b0 + lane_id();
    const u32 v = b < nb ? (part ? part[(u64)b * kt + kk].n : row[b]) : 0u;
    u32 inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const u32 q = __shfl_up_sync(0xffffffffu, inc, o);
      if ((int)lane_id() >= o) inc += q;
    }
    if (b < nb) row[b] = carry + inc - v;
    carry += __shfl_sync(0xffffffffu, inc, 31);
  }
}

__global__ void __launch_bounds__(T3_SC_THREADS)
k_t3_scatter(const u32* __restrict__ kid, const u64* __restrict__ x, u64 n, u32 K, const u32* __restrict__ t3rank,
             u32 n_t3, const u32* __restrict__ n_t3_dev, const u32* __restrict__ off, u64* __restrict__ out) {
  pdl_begin();
  if (n_t3_dev) n_t3 = *n_t3_dev;
  extern __shared__ u32 s_cur[];   // [n_t3]: this block's next output position per segment
  for (u32 t = threadIdx.x; t < n_t3; t += T3_SC_THREADS) s_cur[t] = off[(u64)t * gridDim.x + blockIdx.x];
  __syncthreads();
  u64 r0, r1;
  t3_range(n, gridDim.x, blockIdx.x, &r0, &r1);
  for (u64 i0 = r0 + threadIdx.x; i0 < r1; i0 += (u64)T3_SC_THREADS * T3_U) {
    u32 t[T3_U];
    u64 v[T3_U];
#pragma unroll
    for (int u = 0; u < T3_U; u++) {
      const u64 i = i0 + (u64)u * T3_SC_THREADS;
      t[u] = i < r1 ? __ldcs(kid + i) : 0xFFFFFFFFu;
    }
#pragma unroll
    for (int u = 0; u < T3_U; u++) t[u] = t[u] < K ? __ldg(t3rank + t[u]) : 0xFFFFFFFFu;
    // x only for the Tier-3 rows: a 32-byte sector none of whose rows is Tier-3 is never read
#pragma unroll
    for (int u = 0; u < T3_U; u++) v[u] = t[u] != 0xFFFFFFFFu ? __ldcs(x + i0 + (u64)u * T3_SC_THREADS) : 0ull;
    // only the rows pass A counted (a trace with invalid rows fails after pass A, but these
    // kernels may already run: they must stay inside their ranges)
#pragma unroll
    for (int u = 0; u < T3_U; u++)
      if (t[u] != 0xFFFFFFFFu && v[u] != 0 && v[u] < SIEVE_X_LIMIT) out[atomicAdd(&s_cur[t[u]], 1u)] = v[u];
  }
}

size_t group_t3_temp_bytes(u32 n_t3) { return (size_t)n_t3 * sv_num_sms() * 4 * 4 + 256; }

void launch_group_t3(const u32* kid, const u64* x, u64 n, u32 K, const u32* t3rank, u32 n_t3,
                     const u32* n_t3_dev, const u32* seg_base, u32* cursor, u64* out, void* temp,
                     const KMomPartial* part, int part_grid, u32 part_kt, const u32* t3kern, cudaStream_t s) {
  if (!n || !n_t3) return;
  if (n_t3 <= GT_SMEM_MAX) {
    // pass A's per-block kernel counts over the same row ranges, when the caller has them
    const bool reuse = part && part_grid > 0;
    const u32 nb = reuse ? (u32)part_grid
                         : (u32)std::min<u64>((u64)sv_num_sms() * 4, (n + T3_THREADS - 1) / T3_THREADS);
    u32* cnt = (u32*)temp;   // [n_t3][nb]
    const size_t sm = (size_t)n_t3 * 4;
    sv_smem_attr(k_t3_count, GT_SMEM_MAX * 4);
    sv_smem_attr(k_t3_scatter, GT_SMEM_MAX * 4);
    if (!reuse) SV_LAUNCH(k_t3_count, nb, T3_THREADS, sm, s)(kid, x, n, K, t3rank, n_t3, n_t3_dev, cnt);
    SV_LAUNCH(k_t3_offsets, div_up((u64)n_t3 * 32, 256), 256, 0, s)(cnt, nb, n_t3, n_t3_dev, seg_base,
                                                                    reuse ? part : nullptr, part_kt, t3kern);
    SV_LAUNCH(k_t3_scatter, nb, T3_SC_THREADS, sm, s)(kid, x, n, K, t3rank, n_t3, n_t3_dev, cnt, out);
    return;
  }
  // many Tier-3 kernels: global cursors (k_group_t3's global-atomic branch)
  const u64 tiles = (n + (u64)GR_THREADS * GT_ROWS - 1) / ((u64)GR_THREADS * GT_ROWS);
  const u64 grid = std::min<u64>(tiles, (u64)sv_num_sms() * 2);
  SV_LAUNCH(k_group_t3, (u32)grid, GR_THREADS, 0, s)(kid, x, n, t3rank, n_t3, seg_base, cursor, out);
}

// per chunk: cells (u16) and the chunk's per-cell counts (hist[chunk * G + c]); the counts are
// accumulated two cells per 32-bit word (a chunk holds <= GR_CH < 2^16 values)
__global__ void __launch_bounds__(GR_THREADS)
k_cell_hist(const BucketChunk* __restrict__ chunks, const u64* __restrict__ src, const SegDev* __restrict__ segs,
            u32 G, unsigned short* __restrict__ cells, u32* __restrict__ hist, unsigned long long* inwin) {
  pdl_begin();
  extern __shared__ u32 s_h2[];       // [ceil(G / 2)]
  const BucketChunk ch = chunks[blockIdx.x];
  const u32 gw = (G + 1) / 2;
  for (u32 i = threadIdx.x; i < gw; i += GR_THREADS) s_h2[i] = 0;
  __syncthreads();
  const SegDev g = segs[ch.seg];
  const GridFn gf{__ull2double_rn(g.lo), __uint2double_rn(G - 1), g.hi - g.lo};
  const double w = __dmul_rn(KDE_WC, g.h);
  u64 win = 0;
  u64 xv[GR_CH / GR_THREADS];
#pragma unroll
  for (int q = 0; q < GR_CH / GR_THREADS; q++) {   // the thread's loads first
    const u32 i = threadIdx.x + q * GR_THREADS;
    xv[q] = i < ch.len ? __ldcs(src + ch.begin + i) : 0ull;
  }
#pragma unroll
  for (int q = 0; q < GR_CH / GR_THREADS; q++) {
    const u32 i = threadIdx.x + q * GR_THREADS;
    if (i >= ch.len) continue;
    const u64 x = xv[q];
    unsigned short c = 0xFFFFu;
    if (x >= g.lo && x <= g.hi) {   // a superset range holds a neighbouring part's boundary cell
      // fast path: the estimate is far enough from both neighbouring grid points (SegDev.cm) to
      // decide the cell without evaluating them; else the exact search on the grid
      const double e = __dmul_rn(__ull2double_rn(x - g.lo), g.cq);
      const double jf = floor(e);
      const double f = e - jf;   // exact: e and jf share the binade's ulp grid
      const u32 cc = (f > g.cm && f < 1.0 - g.cm && jf < (double)(G - 1)) ? (u32)jf
                                                                         : cell_arith(gf, G, g.cq, g.lo, x);
      c = (unsigned short)cc;
      atomicAdd(&s_h2[cc >> 1], 1u << (16 * (cc & 1)));
      if (inwin) win += inwin_count(gf, G, g.cq, w, x);
    }
    cells[(u64)blockIdx.x * GR_CH + i] = c;
  }
  __syncthreads();
  u32* hc = hist + (u64)blockIdx.x * G;
  for (u32 c = threadIdx.x; c < G; c += GR_THREADS) hc[c] = (s_h2[c >> 1] >> (16 * (c & 1))) & 0xFFFFu;
  if (inwin) {
    for (int o = 16; o > 0; o >>= 1) win += __shfl_down_sync(0xffffffffu, win, o);
    if (lane_id() == 0 && win) atomicAdd(inwin, (unsigned long long)win);
  }
}

// per (segment s, cell c): rel[chunk * G + c] = values of cell c in the earlier chunks of s,
// tot[s * G + c] = all of them (one thread walks the segment's chunks; consecutive threads read
// consecutive cells of a chunk)
__global__ void k_cell_walk(const u32* __restrict__ seg_chunk, u32 nseg, u32 G, const u32* __restrict__ hist,
                            u32* __restrict__ rel, u32* __restrict__ tot) {
  pdl_begin();
  const u64 id = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= (u64)nseg * G) return;
  const u32 s = (u32)(id / G), c = (u32)(id % G);
  u32 run = 0, k = seg_chunk[s];
  const u32 k1 = seg_chunk[s + 1];
  // eight chunks' counts loaded together (a large segment has thousands of chunks: C5's walk was
  // one dependent load after another, 3.5 ms)
  for (; k + 8 <= k1; k += 8) {
    u32 h[8];
#pragma unroll
    for (int j = 0; j < 8; j++) h[j] = hist[(u64)(k + j) * G + c];
#pragma unroll
    for (int j = 0; j < 8; j++) { rel[(u64)(k + j) * G + c] = run; run += h[j]; }
  }
  for (; k < k1; k++) {
    rel[(u64)k * G + c] = run;
    run += hist[(u64)k * G + c];
  }
  tot[id] = run;
}

// The walk for segments of many chunks, in three parallel steps over groups of <= WALK_GROUP
// chunks (grp[g] = {first chunk, end chunk}, segment s owns groups seg_grp[s] .. seg_grp[s+1]):
// per (group, cell) the group's count; per (segment, cell) the groups' exclusive prefix (in
// place) and the cell total; per (group, cell) the chunks' offsets from the group's prefix.
__global__ void k_walk_gsum(const uint2* __restrict__ grp, u32 ngrp, u32 G, const u32* __restrict__ hist,
                            u32* __restrict__ gs) {
  pdl_begin();
  const u64 id = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= (u64)ngrp * G) return;
  const u32 g = (u32)(id / G), c = (u32)(id % G);
  const uint2 r = grp[g];
  u32 sum = 0, k = r.x;
  for (; k + 8 <= r.y; k += 8) {
    u32 h[8];
#pragma unroll
    for (int j = 0; j < 8; j++) h[j] = hist[(u64)(k + j) * G + c];
#pragma unroll
    for (int j = 0; j < 8; j++) sum += h[j];
  }
  for (; k < r.y; k++) sum += hist[(u64)k * G + c];
  gs[id] = sum;
}
__global__ void k_walk_gscan(const u32* __restrict__ seg_grp, u32 nseg, u32 G, u32* __restrict__ gs,
                             u32* __restrict__ tot) {
  pdl_begin();
  const u64 id = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= (u64)nseg * G) return;
  const u32 s = (u32)(id / G), c = (u32)(id % G);
  u32 run = 0;
  for (u32 g = seg_grp[s]; g < seg_grp[s + 1]; g++) {
    const u32 v = gs[(u64)g * G + c];
    gs[(u64)g * G + c] = run;
    run += v;
  }
  tot[id] = run;
}
__global__ void k_walk_rel(const uint2* __restrict__ grp, u32 ngrp, u32 G, const u32* __restrict__ hist,
                           const u32* __restrict__ gs, u32* __restrict__ rel) {
  pdl_begin();
  const u64 id = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= (u64)ngrp * G) return;
  const u32 g = (u32)(id / G), c = (u32)(id % G);
  const uint2 r = grp[g];
  u32 run = gs[id], k = r.x;
  for (; k + 8 <= r.y; k += 8) {
    u32 h[8];
#pragma unroll
    for (int j = 0; j < 8; j++) h[j] = hist[(u64)(k + j) * G + c];
#pragma unroll
    for (int j = 0; j < 8; j++) { rel[(u64)(k + j) * G + c] = run; run += h[j]; }
  }
  for (; k < r.y; k++) {
    rel[(u64)k * G + c] = run;
    run += hist[(u64)k * G + c];
  }
}

// exclusive prefix of v over a GR_THREADS block; *total receives the block sum
__device__ __forceinline__ u32 block_excl_scan_u32(u32 v, u32* total) {
  __shared__ u32 s_w[GR_THREADS / 32];
  u32 inc = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const u32 t = __shfl_up_sync(0xffffffffu, inc, o);
    if ((int)lane_id() >= o) inc += t;
  }
  const u32 w = threadIdx.x >> 5;
  if (lane_id() == 31) s_w[w] = inc;
  __syncthreads();
  if (w == 0) {
    const u32 t = lane_id() < GR_THREADS / 32 ? s_w[lane_id()] : 0u;
    u32 ti = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const u32 q = __shfl_up_sync(0xffffffffu, ti, o);
      if ((int)lane_id() >= o) ti += q;
    }
    if (lane_id() < GR_THREADS / 32) s_w[lane_id()] = ti - t;
    if (lane_id() == GR_THREADS / 32 - 1) *total = ti;
  }
  __syncthreads();
  const u32 r = s_w[w] + inc - v;
  __syncthreads();
  return r;
}

// per chunk: each value's destination = off[s * G + c] + rel[chunk][c] + its rank among the
// chunk's values of cell c.  The chunk is first staged in shared memory in cell order (local
// positions from a block scan of its counts), then written out so that consecutive threads
// write consecutive addresses of one cell's run.
__global__ void __launch_bounds__(GR_THREADS)
k_cell_scatter(const BucketChunk* __restrict__ chunks, const u64* __restrict__ src,
               const unsigned short* __restrict__ cells, u32 G, const u32* __restrict__ hist,
               const u32* __restrict__ rel, const u32* __restrict__ off, u64* __restrict__ out) {
  pdl_begin();
  extern __shared__ __align__(16) unsigned char smem[];
  u64* s_v = (u64*)smem;                          // [GR_CH]
  unsigned short* s_c = (unsigned short*)(s_v + GR_CH);   // [GR_CH]
  u32* s_ls = (u32*)(s_c + GR_CH);                // [G]: local exclusive scan of the counts
  u32* s_gb = s_ls + G;                           // [G]: global base of the chunk's cell run
  u32* s_cur = s_gb + G;                          // [G]: rank counters
  const BucketChunk ch = chunks[blockIdx.x];
  const u32* hc = hist + (u64)blockIdx.x * G;
  const u32* rc = rel + (u64)blockIdx.x * G;
  const u32* oc = off + (u64)ch.seg * G;
  // block-wide exclusive scan of the G counts (G / GR_THREADS per thread, then the block)
  const u32 per = (G + GR_THREADS - 1) / GR_THREADS;
  const u32 c0 = threadIdx.x * per;
  u32 sum = 0;
  for (u32 c = c0; c < c0 + per && c < G; c++) sum += hc[c];
  __shared__ u32 tot;
  u32 ex = block_excl_scan_u32(sum, &tot);
  for (u32 c = c0; c < c0 + per && c < G; c++) {
    s_ls[c] = ex;
    ex += hc[c];
    s_gb[c] = oc[c] + rc[c];
    s_cur[c] = 0;
  }
  __syncthreads();
  // all of the thread's loads first (GR_CH / GR_THREADS values), then the shared-memory placement
  u64 xv[GR_CH / GR_THREADS];
  unsigned short cv[GR_CH / GR_THREADS];
#pragma unroll
  for (int q = 0; q < GR_CH / GR_THREADS; q++) {
    const u32 i = threadIdx.x + q * GR_THREADS;
    cv[q] = i < ch.len ? cells[(u64)blockIdx.x * GR_CH + i] : (unsigned short)0xFFFFu;
    xv[q] = cv[q] != 0xFFFFu ? __ldcs(src + ch.begin + i) : 0ull;
  }
#pragma unroll
  for (int q = 0; q < GR_CH / GR_THREADS; q++) {
    const unsigned short c = cv[q];
    if (c == 0xFFFFu) continue;
    const u32 p = s_ls[c] + atomicAdd(&s_cur[c], 1u);
    s_v[p] = xv[q];
    s_c[p] = c;
  }
  __syncthreads();
  for (u32 p = threadIdx.x; p < tot; p += GR_THREADS) {
    const u32 c = s_c[p];
    out[s_gb[c] + (p - s_ls[c])] = s_v[p];
  }
}

size_t cell_scatter_smem(u32 G) { return (size_t)GR_CH * 10 + (size_t)G * 12; }

void launch_cell_group(const BucketChunk* chunks, u32 nchunks, const u64* src, const SegDev* segs, u32 nseg,
                       u32 G, const u32* seg_chunk, unsigned short* cells, u32* hist, u32* rel, u32* tot,
                       u32* off, void* scan_temp, u64* out, unsigned long long* inwin, cudaStream_t s,
                       const WalkGroups* wg) {
  const u64 ncell = (u64)nseg * G;
  if (nchunks) {
    const size_t hs = (size_t)(G + 1) / 2 * 4;
    sv_smem_attr(k_cell_hist, (int)hs);
    SV_LAUNCH(k_cell_hist, nchunks, GR_THREADS, hs, s)(chunks, src, segs, G, cells, hist, inwin);
  }
  if (wg && wg->ngrp) {
    const u64 ng = (u64)wg->ngrp * G;
    SV_LAUNCH(k_walk_gsum, div_up(ng, 256), 256, 0, s)(wg->grp, wg->ngrp, G, hist, wg->gs);
    SV_LAUNCH(k_walk_gscan, div_up(ncell, 256), 256, 0, s)(wg->seg_grp, nseg, G, wg->gs, tot);
    SV_LAUNCH(k_walk_rel, div_up(ng, 256), 256, 0, s)(wg->grp, wg->ngrp, G, hist, wg->gs, rel);
  } else {
    SV_LAUNCH(k_cell_walk, div_up(ncell, 256), 256, 0, s)(seg_chunk, nseg, G, hist, rel, tot);
  }
  scan_u32(tot, off, ncell, scan_temp, off + ncell, s);
  if (nchunks) {
    const size_t ss = cell_scatter_smem(G);
    sv_smem_attr(k_cell_scatter, (int)ss);
    SV_LAUNCH(k_cell_scatter, nchunks, GR_THREADS, ss, s)(chunks, src, cells, G, hist, rel, off, out);
  }
}
