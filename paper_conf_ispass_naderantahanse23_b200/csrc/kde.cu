// kde.cu -- fixed-point Gaussian KDE of every open Tier-3 segment on its G-point grid
// ("Kernel Density Estimation [8], [36]"; readings A6-A10 in DESIGN.md section 3):
//
//   g_j  = rn(lo) + rn((hi - lo) * j) / rn(G - 1)                      (A9)
//   z    = rn(rn(g_j - rn(lo)) * inv_h) - rn(rn(x - lo) * inv_h) ;  t = (z * z) * 0.5
//   Q    = 0 if k > 10526, else rint(P(r) * 2^{-j'/256} * 2^(40 - m))   (A10; k = rint(t 256
//          log2 e), j' = k mod 256, m = k div 256, r = t - k rn(ln2/256), P = degree-3 Taylor
//          of e^{-r})
//   D_j  = sum over the segment's values x of Q(x, g_j)   (exact integer sum, u128)
//
// Every floating-point step is an IEEE basic operation written with _rn intrinsics (never
// contracted), so each term is bit-identical to the CPU oracle; the integer sum makes D
// independent of summation order, of the work decomposition and of the number of ranks.
//
// B200 mapping (the paper's scripts have no GPU design; this is new).  The KDE is a windowed
// gather over the values of each segment grouped by grid cell (bucket.cu), bound by the FP64
// pipe (no contraction, so no tensor cores).  Work item = (segment, tile of 32 grid points,
// region of the tile's window |g - x| <= 7.6 h, chunk of <= KDE_CH = 512 values); a region is
// evaluated by the lanes whose windows meet it (32, 16 or 8 lanes with 1, 2 or 4 value slices:
// the staircase of k_kde_tiles); items are dealt to warps round-robin, the last 1/8 claimed from
// a counter as warps finish, and staged by a per-warp cp.async pipeline (see k_kde); each lane owns one grid point and reads the staged values as
// shared-memory broadcasts.  The term is arranged to be
// bit-identical to the oracle's while issuing 9 FP64-pipe instructions and ~6 others:
//   * xs (per value, at staging) and gs (per lane, per item) are the A10 scaled coordinates,
//     so z = gs - xs is one subtraction;
//   * u = z*z replaces t = u/2 (exact scaling): k = nearest integer to u * 128 log2 e (= t * 256
//     log2 e, one rounding, via fma(u, 128 log2 e, 1.5 * 2^52)), r' = u - k rn(ln2)/128 = 2r,
//     Horner on r' with coefficients c_i 2^-i gives exactly the same P (power-of-two scaling
//     commutes with round-to-nearest);
//   * k = low word of that fma result;
//   * S = 2^{-(k mod 256)/256} * 2^(40 - k div 256): a lane-replicated 256-entry table and an
//     exponent-field subtraction (kde_acc); terms with k > 10526 contribute exactly 0;
//   * rint(P * S) = bits(fma(P, S, 2^52)) - bits(2^52): the sum lies in [2^52, 2^53) where the
//     ulp is 1; raw bit patterns are accumulated and 2^52's pattern is subtracted once per term
//     count at the end.
#include <cstdlib>

#include "kernels.cuh"

#define KDE_W 7.6            // window half-width in units of h: k > 10526 (t > 28.5014) beyond it
#define KDE_KCUT 10527       // k > 10526 = rint(28.5 * 256 log2 e) -> index 10527 holds 0
#ifndef KDE_WARPS
#define KDE_WARPS 16         // warps per block (A/B on C4: 16 x 16 terms in flight beat 24 x 8, 28 x 6, 12 x 24)
#endif
#ifndef KDE_MINB
#define KDE_MINB 1           // resident blocks per SM: one 64 KB table shared by the block
#endif
#ifndef KDE_UNROLL
#define KDE_UNROLL 10         // terms in flight per lane (A/B on C4 with the claimed tail: 10 / 12 / 14 / 8
                             // -> 6.01 / 6.11 / 6.19 / 6.22 ms: at 10 and 12 ptxas keeps the accumulators
                             // in place, at 14 it adds five register moves per step; C5 74.0 -> 71.9)
#endif
static_assert(KDE_CH % 32 == 0, "each lane stages KDE_CH / 32 values of an item");
static_assert(KDE_TJ == 32, "a tile is one grid point per lane; narrower shapes are per region");
#define KDE_MAXR 7           // regions per tile (at most 2 * 4 - 1 elementary cell intervals)
#ifndef KDE_ITEM_OVH
#define KDE_ITEM_OVH 64.f    // estimated cost of a work item beyond its terms, in terms per lane
#endif

__device__ __forceinline__ double grid_pt(u64 lo, u64 hi, u32 j, u32 G) {
  return __dadd_rn(__ull2double_rn(lo),
                   __ddiv_rn(__ull2double_rn((hi - lo) * (u64)j), __uint2double_rn(G - 1)));
}

// A region of a tile: a run of whole cells [a, a + len) of the bucketed values and the lanes that
// evaluate it, lanes o .. o + 2^lw - 1 of the tile (grid points j0 + o ...).
struct KdeRegion { u32 a, len, shape; };   // shape = o | lw << 8
static_assert(sizeof(KdeRegion) == 12, "");

// per (segment, tile of 32 grid points): the tile's values split by which lanes need them.
// Lane l needs the cells that meet its window [g_l - 7.6 h, g_l + 7.6 h] (beyond it every term
// is exactly 0).  For each group of m lanes (m = 8, 16 or 32) the cells [L_q, R_q] meet the
// window of some lane of the group; L and R are non-decreasing in q, so the cuts {L_q} U
// {R_q + 1} split the tile's cells into at most 2 * 32/m - 1 intervals, each needed by a
// contiguous run of groups: 8 lanes evaluate it with 4 value slices, 16 lanes with 2 slices,
// 24 or 32 lanes as the whole warp.  Against one 32-lane range per tile the staircase of 8-lane
// steps cuts the out-of-window evaluations at the two ends of the tile's window from
// 2 x 31 x 32 / 2 lane-cells to 2 x 176.  Narrow regions cost extra work items, so the tile
// takes the plan (m = 8, 16 or 32) with the least estimated per-lane cost: terms per lane plus
// `ovh` per work item.  Values a region's lanes do not need (partial cells, the idle group of a
// 3-group interval) are evaluated and add exactly 0, as before.
// One plan (M8 = 4: one 32-lane region; 2: 16-lane steps; 1: 8-lane steps) over the tile's
// per-group cells L[q] (first) and R1[q] (one past the last) and their value offsets LO / RO:
// returns its estimated cost (terms per lane + ovh per work item) and item count, and with EMIT
// writes its regions.  Everything stays in registers (static loops): the cut values are sorted
// with their offsets by a static exchange sort, then each interval between distinct consecutive
// cuts takes the lanes of the groups q with L_q <= p < R1_q (a contiguous run ir .. il - 1);
// adjacent intervals of the same shape merge into one region.
template <int M8, bool EMIT>
__device__ __forceinline__ float kde_tile_plan(const u32 (&L)[4], const u32 (&R1)[4], const u32 (&LO)[4],
                                               const u32 (&RO)[4], u32 ng8, float ovh, u32& items,
                                               KdeRegion* rg) {
  constexpr int NQ = 4 / M8;   // groups of this plan at most
  const u32 ng = (ng8 + M8 - 1) / M8;
  u32 Lm[NQ], Rm[NQ], c[2 * NQ], o[2 * NQ];
#pragma unroll
  for (int q = 0; q < NQ; q++) {
    const bool live = (u32)q < ng;
    const u32 qr = min(ng8 - 1, (u32)(q * M8 + M8 - 1));
    u32 rv = 0, ro = 0;   // R1[qr], RO[qr] by a static select (a dynamic index would spill)
#pragma unroll
    for (int k = 0; k < 4; k++)
      if ((u32)k == qr) { rv = R1[k]; ro = RO[k]; }
    Lm[q] = live ? L[q * M8] : 0xFFFFFFFFu;
    Rm[q] = live ? rv : 0xFFFFFFFFu;
    c[q] = Lm[q]; o[q] = live ? LO[q * M8] : 0u;
    c[NQ + q] = Rm[q]; o[NQ + q] = live ? ro : 0u;
  }
#pragma unroll
  for (int i = 0; i < 2 * NQ; i++)
#pragma unroll
    for (int j = i + 1; j < 2 * NQ; j++)
      if (c[j] < c[i]) {
        const u32 tc = c[i], to = o[i];
        c[i] = c[j]; o[i] = o[j]; c[j] = tc; o[j] = to;
      }
  float cost = 0.f;
  items = 0;
  u32 pa = 0, plen = 0, pshape = 0xFFFFFFFFu, nr = 0;   // the pending region
  auto close = [&]() {
    if (pshape == 0xFFFFFFFFu) return;
    const u32 ni = (plen + KDE_CH - 1) / KDE_CH;
    items += ni;
    cost += (float)plen * (float)(1u << (pshape >> 8)) * (1.f / 32.f) + ovh * (float)ni;
    if (EMIT) { rg[nr].a = pa; rg[nr].len = plen; rg[nr].shape = pshape; }
    nr++;
  };
#pragma unroll
  for (int i = 0; i + 1 < 2 * NQ; i++) {
    const u32 p = c[i], nx = c[i + 1];
    if (nx == 0xFFFFFFFFu || nx == p) continue;
    u32 il = 0, ir = 0;   // groups with L <= p, groups with R1 <= p (both lists non-decreasing)
#pragma unroll
    for (int q = 0; q < NQ; q++) {
      il += Lm[q] <= p;
      ir += Rm[q] <= p;
    }
    if (il <= ir) continue;   // no group needs cells [p, nx)
    const u32 lanes = (il - ir) * 8 * M8;
    const u32 shape = lanes == 8 ? 8 * M8 * ir | 3u << 8 : lanes == 16 ? 8 * M8 * ir | 4u << 8 : 5u << 8;
    const u32 a = o[i], z = o[i + 1];
    if (z <= a) continue;
    if (shape == pshape && pa + plen == a) {
      plen += z - a;
    } else {
      close();
      pa = a; plen = z - a; pshape = shape;
    }
  }
  close();
  if (EMIT)
    for (u32 r = nr; r < KDE_MAXR; r++) rg[r].len = 0;
  return cost;
}

// eight threads per tile: thread (side, q) finds group q's first cell (side 0) or one past its
// last cell (side 1) and that cell's value offset, in parallel (each a short chain of dependent
// loads); the tile's first thread gathers them by shuffles and plans in registers
__global__ void k_kde_tiles(const SegDev* segs, u32 nseg, u32 G, u32 tps, const double* gtab,
                            const u32* off, KdeRegion* regions, u32* tile_items, float ovh) {
  pdl_begin();
  const u64 nt = (u64)nseg * tps;
  const u64 id = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 3;
  const u32 t8 = threadIdx.x & 7, q = t8 & 3, side = t8 >> 2;
  const bool valid = id < nt;
  u32 s = 0, j0 = 0, ng = 0, cell = 0, coff = 0;
  if (valid) {
    s = (u32)(id / tps);
    j0 = (u32)(id % tps) * KDE_TJ;
    ng = (min(G - j0, (u32)KDE_TJ) + 7) / 8;
    if (q < ng) {
      const SegDev g = segs[s];
      const double* gt = gtab + (u64)s * G;
      const double w = __dmul_rn(KDE_W, g.h);
      if (side == 0) {
        const double ga = __dsub_rn(gt[j0 + 8 * q], w);
        const u64 xa = ga <= (double)g.lo ? g.lo : (u64)floor(ga);
        cell = cell_of(gt, G, g.lo, g.cq, xa);
      } else {
        const double gb = __dadd_rn(gt[min(G - 1, j0 + 8 * q + 7)], w);
        const u64 xb = gb >= (double)g.hi ? g.hi : (u64)ceil(gb);
        cell = cell_of(gt, G, g.lo, g.cq, xb) + 1;
      }
      coff = off[(u64)s * G + cell];
    }
  }
  u32 L[4], R1[4], LO[4], RO[4];
  const u32 base = lane_id() & ~7u;
#pragma unroll
  for (int i = 0; i < 4; i++) {
    L[i] = __shfl_sync(0xffffffffu, cell, base + i);
    LO[i] = __shfl_sync(0xffffffffu, coff, base + i);
    R1[i] = __shfl_sync(0xffffffffu, cell, base + 4 + i);
    RO[i] = __shfl_sync(0xffffffffu, coff, base + 4 + i);
  }
  if (!valid || t8 != 0) return;
  KdeRegion* rg = regions + id * KDE_MAXR;
  u32 items = 0, it2 = 0, it1 = 0;
  if (!(ovh < 1e30f)) {   // test hook "inf": one 32-lane region per tile
    kde_tile_plan<4, true>(L, R1, LO, RO, ng, 0.f, items, rg);
    tile_items[id] = items;
    return;
  }
  const float c4 = kde_tile_plan<4, false>(L, R1, LO, RO, ng, ovh, items, rg);
  const float c2 = kde_tile_plan<2, false>(L, R1, LO, RO, ng, ovh, it2, rg);
  const float c1 = kde_tile_plan<1, false>(L, R1, LO, RO, ng, ovh, it1, rg);
  if (c1 < c2 && c1 < c4) kde_tile_plan<1, true>(L, R1, LO, RO, ng, ovh, items, rg);
  else if (c2 < c4) kde_tile_plan<2, true>(L, R1, LO, RO, ng, ovh, items, rg);
  else kde_tile_plan<4, true>(L, R1, LO, RO, ng, ovh, items, rg);
  tile_items[id] = items;
}

size_t kde_region_bytes(u64 ntiles) { return (size_t)ntiles * KDE_MAXR * sizeof(KdeRegion); }
u32 kde_items_per_tile_slack() { return KDE_MAXR - 1; }

// one work item's descriptor, built on the device so a warp can prefetch it with one
// asynchronous 48-byte copy: value range, first grid point and the segment's grid parameters
struct __align__(16) KdeItem {
  u64 va;        // first value (index into the sorted cell keys)
  u32 len;       // values (<= KDE_CH)
  u32 j0;        // grid point of the item's lane 0 (tile start + region offset o)
  u64 lo, hi;    // segment range (grid g_j = rn(lo) + rn((hi - lo) j) / rn(G - 1))
  double inv_h;
  u32 s;         // segment
  unsigned char live;   // lanes with an existing grid point (<= 2^lw)
  unsigned char fast;   // 1: every evaluated |z| < 18.8 (Delta / h < 0.33), so MODE 0 is exact
  unsigned char lw;     // log2 of the lanes per value slice: 5 (32 x 1), 4 (16 x 2), 3 (8 x 4)
  unsigned char pad;
};
static_assert(sizeof(KdeItem) == 48, "KdeItem is copied as three 16-byte pieces");

// item -> descriptor.  Each warp takes a run of consecutive items of the global item space
// (about one run per warp, at most KDE_IT_RUN items, so a large tile's items spread over many
// warps: C5 has tiles of ~1e5 items, which one warp per tile wrote in ~1 ms), finds the tile of
// its first item by a binary search over the scanned counts and walks forward per lane; a lane
// reloads its tile's regions only when its tile changes.  The warp's 32 descriptors of a step
// are staged in shared memory and written as contiguous 16-byte chunks.
#define KDE_IT_RUN 1024
__global__ void k_kde_items(const SegDev* __restrict__ segs, u32 G, u32 tps,
                            const KdeRegion* __restrict__ regions, const u32* __restrict__ tile_items,
                            u32 ntiles, KdeItem* __restrict__ desc) {
  pdl_begin();
  __shared__ __align__(16) KdeItem s_it[8][32];   // blockDim.x = 256
  const u32 lane = lane_id();
  const u32 nwarp = gridDim.x * (blockDim.x >> 5);
  KdeItem* const st = s_it[threadIdx.x >> 5];
  const u32 total = tile_items[ntiles];
  // the KDE's tail-item counter sits right after the last descriptor (the buffer has 16 spare
  // bytes: kde_item_bytes)
  if (blockIdx.x == 0 && threadIdx.x == 0) *(u32*)(desc + total) = 0;
  // runs of a multiple of 32 items, about one per warp (at most KDE_IT_RUN: a larger count
  // takes several passes)
  const u32 run = min((u32)KDE_IT_RUN, max(32u, ((total + nwarp - 1) / nwarp + 31) & ~31u));
  for (u64 base = (u64)(blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * run; base < total;
       base += (u64)nwarp * run) {
    const u32 end = (u32)min((u64)total, base + run);
    // the tile of item `base`: the last tile whose first item is <= base
    u32 lo = 0, hi = ntiles - 1;
    while (lo < hi) {
      const u32 m = (lo + hi + 1) >> 1;
      if (tile_items[m] <= (u32)base) lo = m; else hi = m - 1;
    }
    u32 tile = lo, loaded = 0xFFFFFFFFu, first = 0, s = 0, t = 0;
    KdeRegion R[KDE_MAXR];
    u32 ni[KDE_MAXR];
    SegDev g;
    unsigned char fast = 0;
    for (u32 k0 = (u32)base; k0 < end; k0 += 32) {
      const u32 k = k0 + lane;
      if (k < end) {
        while (tile_items[tile + 1] <= k) tile++;   // tiles are contiguous in the item space
        if (tile != loaded) {
          loaded = tile;
          first = tile_items[tile];
          s = tile / tps;
          t = tile % tps;
          const KdeRegion* rg = regions + (u64)tile * KDE_MAXR;
#pragma unroll
          for (int r = 0; r < KDE_MAXR; r++) {
            R[r] = rg[r];
            ni[r] = (R[r].len + KDE_CH - 1) / KDE_CH;
          }
          g = segs[s];
          // |z| <= 7.6 (window) + 33 grid steps (31 lanes + the two boundary cells) in units of h
          fast = (double)(g.hi - g.lo) < 0.33 * g.h * (double)(G - 1);
        }
        u32 q = k - first, a = 0, len = 0, shape = 0;   // q: the item's chunk inside its region
        bool found = false;
#pragma unroll
        for (int r = 0; r < KDE_MAXR; r++) {      // static selects (no local memory)
          if (!found) {
            if (q < ni[r]) { found = true; a = R[r].a; len = R[r].len; shape = R[r].shape; }
            else q -= ni[r];
          }
        }
        KdeItem d;
        d.va = (u64)a + (u64)q * KDE_CH;
        d.len = min((u32)KDE_CH, len - q * KDE_CH);
        d.j0 = t * KDE_TJ + (shape & 0xFF);
        d.lo = g.lo;
        d.hi = g.hi;
        d.inv_h = g.inv_h;
        d.s = s;
        d.lw = (unsigned char)(shape >> 8);
        d.live = (unsigned char)min(1u << d.lw, G - d.j0);
        d.fast = fast;
        d.pad = 0;
        st[lane] = d;
      }
      __syncwarp();
      const u32 nv = min(32u, end - k0) * 3;   // 16-byte chunks of this step
      const uint4* src = (const uint4*)st;
      uint4* dst = (uint4*)(desc + k0);
      for (u32 c = lane; c < nv; c += 32) dst[c] = src[c];
      __syncwarp();
    }
  }
}

void kde_plan(const SegDev* segs, u32 nseg, u32 G, const double* gtab, const u32* off,
              void* regions, u32* tile_items, void* scan_temp, void* item_desc, cudaStream_t s) {
  u32 tps = div_up(G, KDE_TJ);
  u64 nt = (u64)nseg * tps;
  // SIEVE_KDE_OVH: the per-item cost the plan choice assumes, in terms per lane (A/B and test
  // hook: 0 = always the finest staircase, "inf" = always one 32-lane region per tile)
  const char* e = getenv("SIEVE_KDE_OVH");
  float ovh = e ? (float)atof(e) : KDE_ITEM_OVH;
  if (!(ovh >= 0.f)) ovh = KDE_ITEM_OVH;
  SV_LAUNCH(k_kde_tiles, div_up(nt * 8, 256), 256, 0, s)(segs, nseg, G, tps, gtab, off, (KdeRegion*)regions,
                                                         tile_items, ovh);
  // exclusive scan in place; tile_items[nt] receives the total (read on the device by k_kde)
  scan_u32(tile_items, tile_items, nt, scan_temp, tile_items + nt, s);
  // the work items' descriptors (grids sized by the tiles; the device-side total bounds them)
  SV_LAUNCH(k_kde_items, (u32)sv_num_sms() * 8, 256, 0, s)(segs, G, tps, (const KdeRegion*)regions,
                                                                 tile_items, (u32)nt, (KdeItem*)item_desc);
}

__device__ __forceinline__ void cp_async8(void* sdst, const void* gsrc) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"((u32)__cvta_generic_to_shared(sdst)),
               "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async16(void* sdst, const void* gsrc) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"((u32)__cvta_generic_to_shared(sdst)),
               "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }

// ------------------------------------------------------------------------------------------
#define C_LOG2E_128 0x1.71547652b82fep+7     // 128 * log2(e)  (= the oracle's 256 log2 e / 2)
#define C_LN2_128 0x1.62e42fefa39efp-8      // rn(ln 2) / 128  (= the oracle's rn(ln 2)/256 * 2)
#define C_MAGIC 0x1.8p+52                   // 1.5 * 2^52
#define C_TWO52 0x1.0p+52
// Taylor coefficients of e^{-r} scaled by 2^-i for the argument r' = 2r
#define C_P3 (-0x1.5555555555555p-3 * 0x1p-3)   // rn(-1/6) * 2^-3
#define C_P2 0.125                              //  1/2     * 2^-2
#define C_P1 (-0.5)                             // -1       * 2^-1
#define C_P0 1.0

// 2^(-j/256) correctly rounded for j >= 1; entry 0 is 1 - 2^-53 (A10: no exact ties, see kde_acc)
__constant__ double KDE_EXP2_NEG[256] = {
    0x1.fffffffffffffp-1, 0x1.fe9d96b2a23d9p-1, 0x1.fd3c22b8f71f1p-1, 0x1.fbdba3692d514p-1,
    0x1.fa7c1819e90d8p-1, 0x1.f91d802243c89p-1, 0x1.f7bfdad9cbe14p-1, 0x1.f6632798844f8p-1,
    0x1.f50765b6e4540p-1, 0x1.f3ac948dd7274p-1, 0x1.f252b376bba97p-1, 0x1.f0f9c1cb6412ap-1,
    0x1.efa1bee615a27p-1, 0x1.ee4aaa2188510p-1, 0x1.ecf482d8e67f1p-1, 0x1.eb9f4867cca6ep-1,
    0x1.ea4afa2a490dap-1, 0x1.e8f7977cdb740p-1, 0x1.e7a51fbc74c83p-1, 0x1.e653924676d76p-1,
    0x1.e502ee78b3ff6p-1, 0x1.e3b333b16ee12p-1, 0x1.e264614f5a129p-1, 0x1.e11676b197d17p-1,
    0x1.dfc97337b9b5fp-1, 0x1.de7d5641c0658p-1, 0x1.dd321f301b460p-1, 0x1.dbe7cd63a8315p-1,
    0x1.da9e603db3285p-1, 0x1.d955d71ff6075p-1, 0x1.d80e316c98398p-1, 0x1.d6c76e862e6d3p-1,
    0x1.d5818dcfba487p-1, 0x1.d43c8eacaa1d6p-1, 0x1.d2f87080d89f2p-1, 0x1.d1b532b08c968p-1,
    0x1.d072d4a07897cp-1, 0x1.cf3155b5bab74p-1, 0x1.cdf0b555dc3fap-1, 0x1.ccb0f2e6d1675p-1,
    0x1.cb720dcef9069p-1, 0x1.ca3405751c4dbp-1, 0x1.c8f6d9406e7b5p-1, 0x1.c7ba88988c933p-1,
    0x1.c67f12e57d14bp-1, 0x1.c544778fafb22p-1, 0x1.c40ab5fffd07ap-1, 0x1.c2d1cd9fa652cp-1,
    0x1.c199bdd85529cp-1, 0x1.c06286141b33dp-1, 0x1.bf2c25bd71e09p-1, 0x1.bdf69c3f3a207p-1,
    0x1.bcc1e904bc1d2p-1, 0x1.bb8e0b79a6f1fp-1, 0x1.ba5b030a1064ap-1, 0x1.b928cf22749e4p-1,
    0x1.b7f76f2fb5e47p-1, 0x1.b6c6e29f1c52ap-1, 0x1.b59728de5593ap-1, 0x1.b468415b749b1p-1,
    0x1.b33a2b84f15fbp-1, 0x1.b20ce6c9a8952p-1, 0x1.b0e07298db666p-1, 0x1.afb4ce622f2ffp-1,
    0x1.ae89f995ad3adp-1, 0x1.ad5ff3a3c2774p-1, 0x1.ac36bbfd3f37ap-1, 0x1.ab0e521356ebap-1,
    0x1.a9e6b5579fdbfp-1, 0x1.a8bfe53c12e59p-1, 0x1.a799e1330b358p-1, 0x1.a674a8af46052p-1,
    0x1.a5503b23e255dp-1, 0x1.a42c980460ad8p-1, 0x1.a309bec4a2d33p-1, 0x1.a1e7aed8eb8bbp-1,
    0x1.a0c667b5de565p-1, 0x1.9fa5e8d07f29ep-1, 0x1.9e86319e32323p-1, 0x1.9d674194bb8d5p-1,
    0x1.9c49182a3f090p-1, 0x1.9b2bb4d53fe0dp-1, 0x1.9a0f170ca07bap-1, 0x1.98f33e47a22a2p-1,
    0x1.97d829fde4e50p-1, 0x1.96bdd9a7670b3p-1, 0x1.95a44cbc8520fp-1, 0x1.948b82b5f98e5p-1,
    0x1.93737b0cdc5e5p-1, 0x1.925c353aa2fe2p-1, 0x1.9145b0b91ffc6p-1, 0x1.902fed0282c8ap-1,
    0x1.8f1ae99157736p-1, 0x1.8e06a5e0866d9p-1, 0x1.8cf3216b5448cp-1, 0x1.8be05bad61778p-1,
    0x1.8ace5422aa0dbp-1, 0x1.89bd0a478580fp-1, 0x1.88ac7d98a6699p-1, 0x1.879cad931a436p-1,
    0x1.868d99b4492edp-1, 0x1.857f4179f5b21p-1, 0x1.8471a4623c7adp-1, 0x1.8364c1eb941f7p-1,
    0x1.82589994cce13p-1, 0x1.814d2add106d9p-1, 0x1.80427543e1a12p-1, 0x1.7f3878491c491p-1,
    0x1.7e2f336cf4e62p-1, 0x1.7d26a62ff86f0p-1, 0x1.7c1ed0130c132p-1, 0x1.7b17b0976cfdbp-1,
    0x1.7a11473eb0187p-1, 0x1.790b938ac1cf6p-1, 0x1.780694fde5d3fp-1, 0x1.77024b1ab6e09p-1,
    0x1.75feb564267c9p-1, 0x1.74fbd35d7cbfdp-1, 0x1.73f9a48a58174p-1, 0x1.72f8286ead08ap-1,
    0x1.71f75e8ec5f74p-1, 0x1.70f7466f42e87p-1, 0x1.6ff7df9519484p-1, 0x1.6ef9298593ae5p-1,
    0x1.6dfb23c651a2fp-1, 0x1.6cfdcddd47645p-1, 0x1.6c012750bdabfp-1, 0x1.6b052fa75173ep-1,
    0x1.6a09e667f3bcdp-1, 0x1.690f4b19e9538p-1, 0x1.68155d44ca973p-1, 0x1.671c1c70833f6p-1,
    0x1.6623882552225p-1, 0x1.652b9febc8fb7p-1, 0x1.6434634ccc320p-1, 0x1.633dd1d1929fdp-1,
    0x1.6247eb03a5585p-1, 0x1.6152ae6cdf6f4p-1, 0x1.605e1b976dc09p-1, 0x1.5f6a320dceb71p-1,
    0x1.5e76f15ad2148p-1, 0x1.5d84590998b93p-1, 0x1.5c9268a5946b7p-1, 0x1.5ba11fba87a03p-1,
    0x1.5ab07dd485429p-1, 0x1.59c0827ff07ccp-1, 0x1.58d12d497c7fdp-1, 0x1.57e27dbe2c4cfp-1,
    0x1.56f4736b527dap-1, 0x1.56070dde910d2p-1, 0x1.551a4ca5d920fp-1, 0x1.542e2f4f6ad27p-1,
    0x1.5342b569d4f82p-1, 0x1.5257de83f4eefp-1, 0x1.516daa2cf6642p-1, 0x1.508417f4531eep-1,
    0x1.4f9b2769d2ca7p-1, 0x1.4eb2d81d8abffp-1, 0x1.4dcb299fddd0dp-1, 0x1.4ce41b817c114p-1,
    0x1.4bfdad5362a27p-1, 0x1.4b17dea6db7d7p-1, 0x1.4a32af0d7d3dep-1, 0x1.494e1e192aed2p-1,
    0x1.486a2b5c13cd0p-1, 0x1.4786d668b3237p-1, 0x1.46a41ed1d0057p-1, 0x1.45c2042a7d232p-1,
    0x1.44e086061892dp-1, 0x1.43ffa3f84b9d4p-1, 0x1.431f5d950a897p-1, 0x1.423fb2709468ap-1,
    0x1.4160a21f72e2ap-1, 0x1.40822c367a024p-1, 0x1.3fa4504ac801cp-1, 0x1.3ec70df1c5175p-1,
    0x1.3dea64c123422p-1, 0x1.3d0e544ede173p-1, 0x1.3c32dc313a8e5p-1, 0x1.3b57fbfec6cf4p-1,
    0x1.3a7db34e59ff7p-1, 0x1.39a401b7140efp-1, 0x1.38cae6d05d866p-1, 0x1.37f26231e754ap-1,
    0x1.371a7373aa9cbp-1, 0x1.36431a2de883bp-1, 0x1.356c55f929ff1p-1, 0x1.3496266e3fa2dp-1,
    0x1.33c08b26416ffp-1, 0x1.32eb83ba8ea32p-1, 0x1.32170fc4cd831p-1, 0x1.31432edeeb2fdp-1,
    0x1.306fe0a31b715p-1, 0x1.2f9d24abd886bp-1, 0x1.2ecafa93e2f56p-1, 0x1.2df961f641589p-1,
    0x1.2d285a6e4030bp-1, 0x1.2c57e39771b2fp-1, 0x1.2b87fd0dad990p-1, 0x1.2ab8a66d10f13p-1,
    0x1.29e9df51fdee1p-1, 0x1.291ba7591bb70p-1, 0x1.284dfe1f56381p-1, 0x1.2780e341ddf29p-1,
    0x1.26b4565e27cddp-1, 0x1.25e85711ece75p-1, 0x1.251ce4fb2a63fp-1, 0x1.2451ffb82140ap-1,
    0x1.2387a6e756238p-1, 0x1.22bdda27912d1p-1, 0x1.21f49917ddc96p-1, 0x1.212be3578a819p-1,
    0x1.2063b88628cd6p-1, 0x1.1f9c18438ce4dp-1, 0x1.1ed5022fcd91dp-1, 0x1.1e0e75eb44027p-1,
    0x1.1d4873168b9aap-1, 0x1.1c82f95281c6bp-1, 0x1.1bbe084045cd4p-1, 0x1.1af99f8138a1cp-1,
    0x1.1a35beb6fcb75p-1, 0x1.1972658375d2fp-1, 0x1.18af9388c8deap-1, 0x1.17ed48695bbc0p-1,
    0x1.172b83c7d517bp-1, 0x1.166a45471c3c2p-1, 0x1.15a98c8a58e51p-1, 0x1.14e95934f312ep-1,
    0x1.1429aaea92de0p-1, 0x1.136a814f204abp-1, 0x1.12abdc06c31ccp-1, 0x1.11edbab5e2ab6p-1,
    0x1.11301d0125b51p-1, 0x1.1073028d7233ep-1, 0x1.0fb66affed31bp-1, 0x1.0efa55fdfa9c5p-1,
    0x1.0e3ec32d3d1a2p-1, 0x1.0d83b23395decp-1, 0x1.0cc922b7247f7p-1, 0x1.0c0f145e46c85p-1,
    0x1.0b5586cf9890fp-1, 0x1.0a9c79b1f3919p-1, 0x1.09e3ecac6f383p-1, 0x1.092bdf66607e0p-1,
    0x1.0874518759bc8p-1, 0x1.07bd42b72a836p-1, 0x1.0706b29ddf6dep-1, 0x1.0650a0e3c1f89p-1,
    0x1.059b0d3158574p-1, 0x1.04e5f72f654b1p-1, 0x1.04315e86e7f85p-1, 0x1.037d42e11bbccp-1,
    0x1.02c9a3e778061p-1, 0x1.02168143b0281p-1, 0x1.0163da9fb3335p-1, 0x1.00b1afa5abcbfp-1};

// coefficients without a short (upper-word) immediate form: the constant bank
__constant__ double c_kde[3] = {C_LOG2E_128, C_LN2_128, C_P3};

struct KdeRegs { double log2e, magic; u32 lane8; };  // operands that must sit in registers (see below)

// acc + Q: the term's final fma adds rint(P * S) straight into an integer-valued accumulator in
// [2^52, 2^53) (ulp 1).  rn(acc + P*S) = acc + rint(P*S) exactly because P*S is never an exact
// half-integer: with p, s the odd significands of P and S, P*S = p*s*2^(a+b) has fraction 1/2
// only if a + b = -1, which needs >= 12 trailing zero bits in T_j' (A10 sets T_0 = 1 - 2^-53; the
// other entries have <= 6, pinned in tests), so the sum is exact in any order.
#ifndef KDE_TAIL
#define KDE_TAIL 8           // the last items / KDE_TAIL are claimed dynamically (A/B on C4: 4 / 8 / 16: 6.185 / 6.181 / 6.186 ms against 6.30 all round-robin; 0 = off)
#endif
#ifndef KDE_SPLIT
#define KDE_SPLIT 1          // 1: lane-replicated 256-entry table + exponent arithmetic (below)
#endif
#define KDE_KCLAMP 16383     // KDE_SPLIT: k is clamped here; m = k div 256 <= 63 keeps S normal

// MODE 0: no clamp (the item's |z| < 18.8, so k < 65536 and the byte permutes below see k
// itself; with m = k div 256 <= 255 the scaled entry stays normal); MODE 1: k clamped to
// KDE_KCLAMP; MODE 2: clamp plus the explicit large-u guard (see below).
template <int MODE>
__device__ __forceinline__ double kde_acc(double gs, double xs, const double* sS, KdeRegs R,
                                          double acc) {
  double z = __dsub_rn(gs, xs);                             // A10: both scaled from lo by 1/h
  double u = __dmul_rn(z, z);                               // 2t, exactly
  double kb = __fma_rn(u, R.log2e, R.magic);                // one rounding: nearest integer
  double kf = __dsub_rn(kb, C_MAGIC);
  // k = rint(u * 128 log2 e); any k > 10526 contributes 0.  The low word of kb is k
  // while k < 2^32, i.e. u < 2.3e7: the host proves |z| < 4800 for every (lane, value) pair of
  // a launch when max Delta/h < 140 (window 7.6 h plus KDE_TJ-1 = 31 grid steps plus the two
  // boundary cells of the bucketed range: 7.6 + 33 * 140 < 4800) and runs the
  // unguarded variant; otherwise any u >= 80 is sent to a zero-contribution index explicitly.
  // p stays finite for every input the API admits (x < 2^44, n < 2^36 => h > 2^-26, u < 2^140).
#if KDE_SPLIT
  // S = T'[k] = (2^{-(k mod 256)/256} 2^40) * 2^-(k div 256): the 256-entry table is replicated
  // once per lane (entry e of replica l at byte 256 e + 8 l, so the lanes of every 128-byte
  // wavefront hit distinct bank pairs: conflict-free for any pattern of k), and the power of
  // two is applied exactly in the exponent field.  Two integer instructions besides the load:
  //   * one byte permute gives the replica address (k mod 256) << 8 | 8 l (the table sits at
  //     the start of shared memory, so the load takes no base register);
  //   * the replica stores entry e with e << 12 added to its upper word, so one multiply-add
  //     hi - k * 2^12 = hi(2^{-e/256} 2^40) - (k div 256) * 2^20 (k = 256 (k div 256) + e; the
  //     upper word never wraps: k < 2^16) applies the power of two.
  // For 10526 < k <= KDE_KCLAMP, P * S <= 1.0014 * 2^(40 - 10527/256) < 0.47, so
  // fma(P, S, acc) = acc exactly: the term is 0 as A10 defines, with no select.
  u32 k = (u32)__double2loint(kb);
  if (MODE >= 1) k = min(k, (u32)KDE_KCLAMP);
  if (MODE == 2) k = (u32)__double2hiint(u) >= 0x40540000u ? (u32)KDE_KCLAMP : k;
  double T = *(const double*)((const char*)sS + __byte_perm(k, R.lane8, 0x5504u));
  double S = __hiloint2double(__double2hiint(T) - (int)(k << 12), __double2loint(T));
#else
  // fma(p, 0, acc) = acc for the zero entry T'[KDE_KCUT]
  u32 k = min((u32)__double2loint(kb), (u32)KDE_KCUT);
  if (MODE == 2) k = (u32)__double2hiint(u) >= 0x40540000u ? (u32)KDE_KCUT : k;
  double S = sS[k];
#endif
  double r = __fma_rn(-kf, c_kde[1], u);
  double p = __fma_rn(c_kde[2], r, C_P2);
  p = __fma_rn(p, r, C_P1);
  p = __fma_rn(p, r, C_P0);
  return __fma_rn(p, S, acc);
}

#if KDE_SPLIT
#define KDE_SMEM_TABLE (256 * 32 * 8)
#else
#define KDE_SMEM_TABLE ((KDE_KCUT + 1) * 8)
#endif
// one lane's sum over the item's values: KDE_UNROLL independent accumulators, each an integer
// in [2^52, 2^53) (a lane adds at most KDE_CH terms of <= 2^40 per item)
// pair of staged values at a shared-memory byte address (a 128-bit shared load); volatile with a
// memory clobber so the compiler keeps it behind the staging stores and __syncwarp
__device__ __forceinline__ double2 lds_f64x2(u32 addr) {
  double2 v;
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(addr) : "memory");
  return v;
}

// one lane's run of len staged values starting at the shared-memory byte address sa (16-byte
// aligned: runs start at even indices), read as 128-bit pairs with one induction variable
template <int MODE>
__device__ __forceinline__ u64 kde_run_sum(double gs, u32 sa, u32 len, const double* sSb, KdeRegs R) {
  static_assert(KDE_UNROLL % 2 == 0, "values are loaded in pairs");
  double ac[KDE_UNROLL];
#pragma unroll
  for (int q = 0; q < KDE_UNROLL; q++) ac[q] = C_TWO52;
  const u32 steps = len / KDE_UNROLL;   // full steps; the rest (< KDE_UNROLL values) one by one
  const u32 ea = sa + steps * (KDE_UNROLL * 8);
  u32 a = sa;
  for (; a != ea; a += KDE_UNROLL * 8) {
#pragma unroll
    for (int q = 0; q < KDE_UNROLL / 2; q++) {
      const double2 v = lds_f64x2(a + 16 * q);
      ac[2 * q] = kde_acc<MODE>(gs, v.x, sSb, R, ac[2 * q]);
      ac[2 * q + 1] = kde_acc<MODE>(gs, v.y, sSb, R, ac[2 * q + 1]);
    }
  }
  const u32 rest = len - steps * KDE_UNROLL;   // < KDE_UNROLL
#pragma unroll
  for (int q = 0; q < KDE_UNROLL - 1; q++) {
    if ((u32)q < rest) {
      double v;
      asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a + 8 * q) : "memory");
      ac[q] = kde_acc<MODE>(gs, v, sSb, R, ac[q]);
    }
  }
  u64 acc = 0;
#pragma unroll
  for (int q = 0; q < KDE_UNROLL; q++) acc += (u64)__double_as_longlong(ac[q]) - 0x4330000000000000ull;
  return acc;
}

// per warp: two value buffers (double-buffered asynchronous staging) and a ring of three item
// descriptors (current, next, the one after)
#define KDE_WARP_BYTES (2 * KDE_CH * 8 + 3 * 48)
#define KDE_SMEM_BYTES (KDE_SMEM_TABLE + KDE_WARPS * KDE_WARP_BYTES)

// A warp evaluates one item: its 2^lw lanes-per-slice own grid points j0 .. j0 + 2^lw - 1 (lane
// l: j0 + l mod 2^lw) and the 32 / 2^lw value slices split the item's values into contiguous
// runs (slice l div 2^lw); slices are summed with shuffles.  Whole-warp items (lw = 5) are the
// tile's core, narrower ones the staircase at the ends of its window (k_kde_tiles).
//
// Items are dealt to warps round-robin (item w, w + W, w + 2W, ...; W warps in the grid) up to the
// last items / KDE_TAIL, which warps claim from a counter as they run out (so the SMs finish
// together); every warp knows its next two items, and a three-stage cp.async pipeline keeps all
// global latency off the FP64 pipe: while item k is evaluated, the values of item k + 1 and the
// descriptor of item k + 2 are in flight.  Densities are accumulated with fire-and-forget
// reductions of two limbs (low 32 bits, the rest) into D[2j], D[2j + 1]; k_valleys turns them
// into the u128 D_j.
#if KDE_TAIL
// the warp's next item from the tail counter (lane 0 claims, the warp shares it); kept out of line
// so the claim does not enter the register allocation of the term loop
__device__ __noinline__ u32 kde_claim_tail(const KdeItem* desc, u32 items) {
  const u32 S = items - items / KDE_TAIL;
  u32 c = 0;
  if (lane_id() == 0) c = atomicAdd((u32*)(desc + items), 1u);
  c = __shfl_sync(0xffffffffu, c, 0);
  return S + c < items ? S + c : items;
}
#endif

template <bool GUARD>
__global__ void __launch_bounds__(32 * KDE_WARPS, KDE_MINB)
k_kde(const KdeItem* __restrict__ desc, const u32* __restrict__ n_items, u32 G,
      const u64* __restrict__ vals, u32 vshift, u64* D, unsigned long long* evaluated,
      bool allow_fast) {
  pdl_begin();
  extern __shared__ __align__(16) unsigned char smem[];
  double* sS = (double*)smem;
#if KDE_SPLIT
  // replica l of entry e at double index 32 e + l: 2^{-e/256} * 2^40 (exact scaling), its upper
  // word biased by e << 12 for kde_acc's exponent step
  for (u32 q = threadIdx.x; q < 256 * 32; q += blockDim.x) {
    double T = KDE_EXP2_NEG[q >> 5];
    sS[q] = __hiloint2double(__double2hiint(T) + 40 * (1 << 20) + (int)((q >> 5) << 12), __double2loint(T));
  }
#else
  // T'[k] = ldexp(2^{-(k mod 256)/256}, 40 - k div 256), T'[KCUT] = 0
  for (u32 k = threadIdx.x; k <= KDE_KCUT; k += blockDim.x) {
    double T = KDE_EXP2_NEG[k & 255];
    sS[k] = k == KDE_KCUT ? 0.0
                          : __hiloint2double(__double2hiint(T) + (40 - (int)(k >> 8)) * (1 << 20),
                                             __double2loint(T));
  }
#endif
  __syncthreads();  // the last block-wide barrier: warps run independently from here
  const u32 items = *n_items;  // device-side total of work items
  const u32 lane = lane_id();
  const u32 W = gridDim.x * KDE_WARPS;
  u32 it = blockIdx.x * KDE_WARPS + (threadIdx.x >> 5);
  if (it >= items) return;
#if KDE_TAIL
  // a warp whose first round-robin item lies in the claimed tail claims its first item instead
  // (every tail item is handed out exactly once, by the counter)
  if (it >= items - items / KDE_TAIL) {
    it = kde_claim_tail(desc, items);
    if (it >= items) return;
  }
#endif
  unsigned char* wsm = smem + KDE_SMEM_TABLE + (threadIdx.x >> 5) * KDE_WARP_BYTES;
  double* const buf0 = (double*)wsm;   // value buffers buf0 + b * KDE_CH, b = 0, 1
  KdeItem* sd = (KdeItem*)(wsm + 2 * KDE_CH * 8);
  const double* sSb = sS;   // KDE_SPLIT: the lane's replica is selected by R.lane8
  KdeRegs R;
  R.lane8 = 8 * lane;
  // the fma that forms kb has two constant operands and a DFMA takes at most one constant:
  // load both into registers once (opaque to the compiler, so it cannot re-materialise them)
  asm volatile("mov.b64 %0, %1;" : "=d"(R.log2e) : "d"(c_kde[0]));
  asm volatile("mov.b64 %0, %1;" : "=d"(R.magic) : "d"(C_MAGIC));

  auto fetch_desc = [&](u32 item, KdeItem* dst) {
    if (lane < 3) cp_async16((char*)dst + 16 * lane, (const char*)(desc + item) + 16 * lane);
  };
  auto fetch_vals = [&](const KdeItem* d, double* dst) {
    const u64* src = vals + d->va;
    const u32 len = d->len;
#pragma unroll
    for (u32 q = 0; q < KDE_CH / 32; q++) {
      const u32 i = lane + 32 * q;
      if (i < len) cp_async8(dst + i, src + i);
    }
  };
  // prologue: descriptor of the first item, then its values and the second item's descriptor
  fetch_desc(it, sd);
  cp_async_commit();
  cp_async_wait_all();
  __syncwarp();
  fetch_vals(sd, buf0);
#if KDE_TAIL
  // Items below S = items - items / KDE_TAIL are dealt round-robin; the last items / KDE_TAIL are
  // claimed from a counter (desc + items, zeroed by k_kde_items), so the SMs that drew cheaper
  // items take more of the tail and finish with the others.
  auto next_of = [&](u32 cur_it) -> u32 {   // the item after cur_it for this warp
    if (cur_it >= items) return items;
    if (cur_it + W < items - items / KDE_TAIL) return cur_it + W;
    return kde_claim_tail(desc, items);
  };
  u32 nx1 = next_of(it);
  if (nx1 < items) fetch_desc(nx1, sd + 1);
#else
  if (it + W < items) fetch_desc(it + W, sd + 1);
#endif
  cp_async_commit();
  u32 cur = 0, b = 0;   // ring slot of the current descriptor, current value buffer
  for (;;) {
    cp_async_wait_all();  // values of this item, descriptor of the next (issued one item ago)
    __syncwarp();
    const KdeItem* cd = sd + cur;
    const u32 nxt = cur == 2 ? 0 : cur + 1, nn = nxt == 2 ? 0 : nxt + 1;
#if KDE_TAIL
    const u32 it1 = nx1;
    const u32 it2 = next_of(it1);
    if (it1 < items) {
      fetch_vals(sd + nxt, buf0 + (b ^ 1) * KDE_CH);
      if (it2 < items) fetch_desc(it2, sd + nn);
    }
    nx1 = it2;
#else
    const u32 it1 = it + W;
    if (it1 < items) {
      fetch_vals(sd + nxt, buf0 + (b ^ 1) * KDE_CH);
      if (it1 + W < items) fetch_desc(it1 + W, sd + nn);
    }
#endif
    cp_async_commit();
    double* sx = buf0 + b * KDE_CH;
    const u32 len = cd->len;
    // each lane converts the values it copied itself: x = key >> vshift (lo <= x <= hi), then
    // xs = rn(rn(x - lo) * inv_h) (A10; x - lo is an exact integer below 2^44)
    const u64 lo = cd->lo;
    const double inv_h = cd->inv_h;
#pragma unroll
    for (u32 q = 0; q < KDE_CH / 32; q++) {
      const u32 i = lane + 32 * q;
      if (i < len)
        sx[i] = __dmul_rn(__ull2double_rn(((u64)__double_as_longlong(sx[i]) >> vshift) - lo), inv_h);
    }
    __syncwarp();
    const u32 lw = cd->lw;
    const u32 slice = lane >> lw;
    const u32 j = cd->j0 + (lane & ((1u << lw) - 1u));
    // the slice's values: runs of an even length cs (16-byte aligned), cs != 0 mod 8 so the (up
    // to four) slices' 128-bit loads fall in different banks
    u32 cs = ((len >> (5 - lw)) + 2) & ~1u;
    if ((cs & 7u) == 0) cs += 2;
    const u32 sa = min(len, slice * cs);
    const u32 sn = min(len - sa, cs);
    // gs = rn(rn(g_j - rn(lo)) * inv_h) (A10)
    const double gs = __dmul_rn(__dsub_rn(grid_pt(lo, cd->hi, j < G ? j : G - 1, G), __ull2double_rn(lo)), inv_h);
    const bool fast = !GUARD && allow_fast && cd->fast;
    const u32 ra = (u32)__cvta_generic_to_shared(sx + sa);
    u64 acc = fast ? kde_run_sum<0>(gs, ra, sn, sSb, R) : kde_run_sum<GUARD ? 2 : 1>(gs, ra, sn, sSb, R);
    for (u32 o = 1u << lw; o < 32; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    // evaluated (lane, value) pairs of this item, wasted ones included
    if (evaluated && lane == 0) atomicAdd(evaluated, (unsigned long long)cd->live * len);
    if (j < G && slice == 0 && acc) {
      unsigned long long* d = (unsigned long long*)(D + 2 * ((u64)cd->s * G + j));
      atomicAdd(d, acc & 0xFFFFFFFFull);                 // < 2^32 items per grid point: exact
      if (acc >> 32) atomicAdd(d + 1, acc >> 32);
    }
    __syncwarp();  // buffer b and descriptor slot cur are refilled from the next iteration on
    it = it1;
    if (it >= items) break;
    cur = nxt;
    b ^= 1;
  }
}

// D[2j] (sum of low 32-bit limbs), D[2j + 1] (sum of high parts) -> u128 D_j
__global__ void k_kde_fix(u64* D, u64 n) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  u64 lo = D[2 * i], hi = D[2 * i + 1];
  u64 l = lo + (hi << 32);
  D[2 * i] = l;
  D[2 * i + 1] = (hi >> 32) + (l < lo);
}

size_t kde_item_bytes(u32 items) { return (size_t)items * sizeof(KdeItem) + 16; }

void launch_kde(const SegDev* segs, u32 nseg, u32 G, const u64* vals, u32 vshift, const void* regions,
                const u32* tile_items, void* item_desc, u32 items, u64* D,
                unsigned long long* evaluated, bool guard, bool fix, cudaStream_t s) {
  if (items == 0) {
    if (fix) launch_kde_fix(D, (u64)nseg * G, s);
    return;
  }
  u32 tps = div_up(G, KDE_TJ);
  u32 ntiles = nseg * tps;
  // `items` is a host-side upper bound: grids are sized by it, the kernels stop at the
  // device-side count tile_items[ntiles]
  KdeItem* desc = (KdeItem*)item_desc;   // written by kde_plan
  // test hook SIEVE_KDE_FORCE: 1 = never the unclamped fast path, 2 = always the guarded
  // variant (all three evaluate identical terms; the parity tests run each)
  const char* force = getenv("SIEVE_KDE_FORCE");
  const int fm = force ? atoi(force) : 0;
  if (fm >= 2) guard = true;
  auto kern = guard ? k_kde<true> : k_kde<false>;
  sv_smem_attr(kern, KDE_SMEM_BYTES);
  static int occ[2][64];  // resident blocks per SM, per variant and device (queried once)
  int dev = 0;
  cudaGetDevice(&dev);
  int& per_sm = occ[guard][dev & 63];
  if (per_sm < 1) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 32 * KDE_WARPS, KDE_SMEM_BYTES);
    if (per_sm < 1) per_sm = 1;
  }
  u32 grid = (u32)sv_num_sms() * (u32)per_sm;
  u32 need = div_up(items, KDE_WARPS);
  if (grid > need) grid = need;
  SV_LAUNCH(kern, grid, 32 * KDE_WARPS, KDE_SMEM_BYTES, s)(desc, tile_items + ntiles, G, vals, vshift, D,
                                                           evaluated, fm == 0);
  if (fix) launch_kde_fix(D, (u64)nseg * G, s);
}

void launch_kde_fix(u64* D, u64 npoints, cudaStream_t s) {
  if (npoints) SV_LAUNCH(k_kde_fix, div_up(npoints, 256), 256, 0, s)(D, npoints);
}
