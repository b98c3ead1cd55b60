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
    for (u64 i = i0 + threadIdx.x; i < i1; i += PS_THREADS) {
      u64 x = vals[i] >> vshift;
      if (x >= a && x < b) {
        n++;
        add128(s1lo, s1hi, x, 0);
        add128(s2lo, s2hi, x * x, __umul64hi(x, x));
        mn = x < mn ? x : mn;
        mx = x > mx ? x : mx;
      }
    }
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
__global__ void k_part_pack(const u32* __restrict__ part_off, u32 nseg, u32 cap, const u64* __restrict__ lanes,
                            const u64* __restrict__ mm, const u64* __restrict__ ab, u64* out) {
  const u32 nparts = part_off[nseg];
  u32 p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p == 0) out[0] = nparts;
  if (p >= nparts) return;
  u64* o = out + 1 + (u64)p * PART_REC;
  for (int k = 0; k < MOM_LANES; k++) o[k] = lanes[(u64)p * MOM_LANES + k];
  o[MOM_LANES] = mm[p];
  o[MOM_LANES + 1] = mm[cap + p];
  o[MOM_LANES + 2] = ab[4 * (u64)p + 2];
  o[MOM_LANES + 3] = ab[4 * (u64)p + 3];
}

void launch_part_pack(const u32* part_off, u32 nseg, u32 cap, const u64* lanes, const u64* mm,
                      const u64* ab, u64* out, cudaStream_t s) {
  SV_LAUNCH(k_part_pack, div_up(std::max<u32>(cap, 1), 128), 128, 0, s)(part_off, nseg, cap, lanes, mm, ab, out);
}
