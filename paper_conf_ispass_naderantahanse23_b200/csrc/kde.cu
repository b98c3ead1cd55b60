// kde.cu -- fixed-point Gaussian KDE of every open Tier-3 segment on its G-point grid
// ("Kernel Density Estimation [8], [36]"; readings A6-A10 in DESIGN.md section 3):
//
//   g_j  = rn(lo) + rn((hi - lo) * j) / rn(G - 1)                      (A9)
//   z    = (g_j - rn(x)) * inv_h ;  t = (z * z) * 0.5
//   Q    = 0 if t > 37, else rint(P(r) * 2^{-j'/64} * 2^(52 - m))    (A10; k = rint(t 64 log2 e),
//          j' = k mod 64, m = k div 64, r = t - k ln2/64, P = degree-5 Taylor of e^{-r})
//   D_j  = sum over the segment's values x of Q(x, g_j)   (exact integer sum, u128)
//
// Every floating-point step is an IEEE basic operation written with _rn intrinsics (never
// contracted), so each term is bit-identical to the CPU oracle; the integer sum makes D
// independent of summation order, of the work decomposition and of the number of ranks.
//
// B200 mapping (the paper's scripts have no GPU design; this is new).  The KDE is a windowed
// gather over the SORTED values of each segment, bound by the FP64 pipe (no contraction, so no
// tensor cores).  Work item = (segment, tile of 32 grid points, chunk of <= 256 values inside
// the tile's window |g - x| <= 8.7 h); items are pulled by WARPS from an atomic counter (no
// block barriers: warps of a block never wait for each other); each lane owns one grid point,
// the chunk is staged in the warp's slice of shared memory and read as broadcasts.  The term is
// arranged to be bit-identical to the oracle's while issuing 13 FP64-pipe instructions and ~6
// others:
//   * u = z*z replaces t = u/2 (exact scaling): k = nearest integer to u * 32 log2 e (= t * 64
//     log2 e, one rounding, via fma(u, 32 log2 e, 1.5 * 2^52)), r' = u - k ln2/32 = 2r,
//     Horner on r' with coefficients c_i 2^-i gives exactly the same P (power-of-two scaling
//     commutes with round-to-nearest);
//   * k = low word of that fma result, clamped to 3417;
//   * S = T'[k] = 2^{-(k mod 64)/64} * 2^(52 - k div 64) from a shared-memory table (exact
//     power-of-two scalings of the correctly rounded 2^{-j/64}), with T'[3417] = 0: every
//     t > 37 lands on k >= 3417 or has Q = 0 anyway (e^-37 2^52 = 0.38), so no select;
//   * rint(P * S) = bits(fma(P, S, 2^52)) - bits(2^52): the sum lies in [2^52, 2^53] where the
//     ulp is 1; raw bit patterns are accumulated and 2^52's pattern is subtracted once per term
//     count at the end.
#include "kernels.cuh"

#define KDE_W 8.7            // window half-width in units of h: t > 37 is guaranteed beyond it
#define KDE_WC 8.602325267042627  // sqrt(74): |z| <= this <=> t <= 37 (term-count diagnostic)
#define KDE_KCUT 3417        // rint(37 * 64 log2 e) = 3416; index 3417 holds 0
#ifndef KDE_WARPS
#define KDE_WARPS 8          // warps per block (independent work-item consumers)
#endif
#ifndef KDE_MINB
#define KDE_MINB 3           // min resident blocks per SM (register budget: 85 / thread)
#endif
#ifndef KDE_UNROLL
#define KDE_UNROLL 8         // terms in flight per lane
#endif
#define KDE_V (32 / KDE_TJ)  // value slices per warp

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

// per (segment, tile of KDE_TJ grid points): the local index range of the values inside the
// tile's window, and the number of KDE_CH-value chunks (work items) it takes
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
  // exclusive scan in place; tile_items[nt] receives the total (read on the device by k_kde)
  scan_u32(tile_items, tile_items, nt, scan_temp, tile_items + nt, s);
  if (items_host) {
    SV_CUDA(cudaMemcpyAsync(items_host, tile_items + nt, 4, cudaMemcpyDeviceToHost, s));
    SV_CUDA(cudaStreamSynchronize(s));
  }
  return SIEVE_OK;
}

// item -> tile map (so a warp finds its tile with one load): one thread per item, binary
// search of the last tile whose first item is <= it
__global__ void k_kde_items(const u32* tile_items, u32 ntiles, u32* item_tile) {
  const u32 items = tile_items[ntiles];  // device-side total (no host round trip)
  for (u32 it = blockIdx.x * blockDim.x + threadIdx.x; it < items; it += gridDim.x * blockDim.x) {
    u32 lo = 0, hi = ntiles - 1;
    while (lo < hi) {
      u32 m = (lo + hi + 1) >> 1;
      if (tile_items[m] <= it) lo = m; else hi = m - 1;
    }
    item_tile[it] = lo;
  }
}

// ------------------------------------------------------------------------------------------
#define C_LOG2E_32 0x1.71547652b82fep+5     // 32 * log2(e)  (= the oracle's 64 log2 e / 2)
#define C_LN2_32_HI 0x1.62e42fee00000p-6    // ln2/32 high part (21 significant bits)
#define C_LN2_32_LO 0x1.a39ef35793c76p-38
#define C_MAGIC 0x1.8p+52                   // 1.5 * 2^52
#define C_TWO52 0x1.0p+52
// Taylor coefficients of e^{-r} scaled by 2^-i for the argument r' = 2r
#define C_P5 (-0x1.1111111111111p-7 * 0x1p-5)   // -1/120 * 2^-5
#define C_P4 (0x1.5555555555555p-5 * 0x1p-4)    //  1/24  * 2^-4
#define C_P3 (-0x1.5555555555555p-3 * 0x1p-3)   // -1/6   * 2^-3
#define C_P2 0.125                              //  1/2   * 2^-2
#define C_P1 (-0.5)                             // -1     * 2^-1
#define C_P0 1.0

__constant__ double KDE_EXP2_NEG[64] = {
    0x1.0000000000000p+0, 0x1.fa7c1819e90d8p-1, 0x1.f50765b6e4540p-1, 0x1.efa1bee615a27p-1,
    0x1.ea4afa2a490dap-1, 0x1.e502ee78b3ff6p-1, 0x1.dfc97337b9b5fp-1, 0x1.da9e603db3285p-1,
    0x1.d5818dcfba487p-1, 0x1.d072d4a07897cp-1, 0x1.cb720dcef9069p-1, 0x1.c67f12e57d14bp-1,
    0x1.c199bdd85529cp-1, 0x1.bcc1e904bc1d2p-1, 0x1.b7f76f2fb5e47p-1, 0x1.b33a2b84f15fbp-1,
    0x1.ae89f995ad3adp-1, 0x1.a9e6b5579fdbfp-1, 0x1.a5503b23e255dp-1, 0x1.a0c667b5de565p-1,
    0x1.9c49182a3f090p-1, 0x1.97d829fde4e50p-1, 0x1.93737b0cdc5e5p-1, 0x1.8f1ae99157736p-1,
    0x1.8ace5422aa0dbp-1, 0x1.868d99b4492edp-1, 0x1.82589994cce13p-1, 0x1.7e2f336cf4e62p-1,
    0x1.7a11473eb0187p-1, 0x1.75feb564267c9p-1, 0x1.71f75e8ec5f74p-1, 0x1.6dfb23c651a2fp-1,
    0x1.6a09e667f3bcdp-1, 0x1.6623882552225p-1, 0x1.6247eb03a5585p-1, 0x1.5e76f15ad2148p-1,
    0x1.5ab07dd485429p-1, 0x1.56f4736b527dap-1, 0x1.5342b569d4f82p-1, 0x1.4f9b2769d2ca7p-1,
    0x1.4bfdad5362a27p-1, 0x1.486a2b5c13cd0p-1, 0x1.44e086061892dp-1, 0x1.4160a21f72e2ap-1,
    0x1.3dea64c123422p-1, 0x1.3a7db34e59ff7p-1, 0x1.371a7373aa9cbp-1, 0x1.33c08b26416ffp-1,
    0x1.306fe0a31b715p-1, 0x1.2d285a6e4030bp-1, 0x1.29e9df51fdee1p-1, 0x1.26b4565e27cddp-1,
    0x1.2387a6e756238p-1, 0x1.2063b88628cd6p-1, 0x1.1d4873168b9aap-1, 0x1.1a35beb6fcb75p-1,
    0x1.172b83c7d517bp-1, 0x1.1429aaea92de0p-1, 0x1.11301d0125b51p-1, 0x1.0e3ec32d3d1a2p-1,
    0x1.0b5586cf9890fp-1, 0x1.0874518759bc8p-1, 0x1.059b0d3158574p-1, 0x1.02c9a3e778061p-1};

// coefficients without a short (upper-word) immediate form: the constant bank
__constant__ double c_kde[6] = {C_LOG2E_32, C_LN2_32_HI, C_LN2_32_LO, C_P5, C_P4, C_P3};

struct KdeRegs { double log2e, magic; };  // operands that must sit in registers (see below)

// raw bit pattern of fma(P, S, 2^52); the term is this minus bits(2^52)
template <bool GUARD>
__device__ __forceinline__ u64 kde_qbits(double g, double xd, double inv_h, const double* sS,
                                         KdeRegs R) {
  double z = __dmul_rn(__dsub_rn(g, xd), inv_h);
  double u = __dmul_rn(z, z);                               // 2t, exactly
  double kb = __fma_rn(u, R.log2e, R.magic);                // one rounding: nearest integer
  double kf = __dsub_rn(kb, C_MAGIC);
  // k = rint(u * 32 log2 e); any k >= 3417 (t > 37) maps to the zero entry.  The low word of kb
  // is k while k < 2^32, i.e. u < 9.3e7: the host proves |z| < 9645 for every (lane, value)
  // pair of a launch when max Delta/h < 300 (window 8.7 h plus KDE_TJ-1 = 31 grid steps) and
  // runs the unguarded variant; otherwise any u >= 80 is sent to the zero entry explicitly.  p
  // stays finite for every input the API admits (x < 2^44, n < 2^36 => h > 2^-26, u < 2^140),
  // and fma(p, 0, 2^52) = 2^52.
  u32 k = min((u32)__double2loint(kb), (u32)KDE_KCUT);
  if (GUARD) k = (u32)__double2hiint(u) >= 0x40540000u ? (u32)KDE_KCUT : k;
  double r = __fma_rn(-kf, c_kde[1], u);
  r = __fma_rn(-kf, c_kde[2], r);
  double p = __fma_rn(c_kde[3], r, c_kde[4]);
  p = __fma_rn(p, r, c_kde[5]);
  p = __fma_rn(p, r, C_P2);
  p = __fma_rn(p, r, C_P1);
  p = __fma_rn(p, r, C_P0);
  return (u64)__double_as_longlong(__fma_rn(p, sS[k], C_TWO52));
}

#define KDE_SMEM_TABLE ((KDE_KCUT + 1) * 8)
#define KDE_SMEM_BYTES (KDE_SMEM_TABLE + KDE_WARPS * KDE_CH * 8)

// A warp owns KDE_TJ grid points x KDE_V = 32 / KDE_TJ value slices: lane l evaluates grid
// point j0 + l % KDE_TJ over the values i = l / KDE_TJ + m * KDE_V; slices are summed with
// shuffles.  (Measured: 32 x 1 beats 8 x 4 -- the narrower value window of 8 x 4 saves ~10%
// out-of-window terms but quadruples the per-item overhead at equal chunk size.)
template <bool GUARD>
__global__ void __launch_bounds__(32 * KDE_WARPS, KDE_MINB)
k_kde(const SegDev* __restrict__ segs, u32 G, u32 tps, const u64* __restrict__ keys, u64 xmask,
      const u64* __restrict__ tile_range, const u32* __restrict__ tile_items,
      const u32* __restrict__ item_tile, u32 ntiles, u64* D, unsigned long long* counter,
      unsigned long long* terms) {
  const u32 items = tile_items[ntiles];  // device-side total of work items
  extern __shared__ __align__(16) unsigned char smem[];
  double* sS = (double*)smem;                                   // [KDE_KCUT + 1]
  double* sx = (double*)(smem + KDE_SMEM_TABLE) + (threadIdx.x >> 5) * KDE_CH;  // warp's slice
  // T'[k] = ldexp(2^{-(k mod 64)/64}, 52 - k div 64), T'[KCUT] = 0
  for (u32 k = threadIdx.x; k <= KDE_KCUT; k += blockDim.x) {
    double T = KDE_EXP2_NEG[k & 63];
    sS[k] = k == KDE_KCUT ? 0.0
                          : __hiloint2double(__double2hiint(T) + (int)((52u - (k >> 6)) << 20),
                                             __double2loint(T));
  }
  __syncthreads();
  const u32 lane = lane_id();
  u64 inwin = 0;
  // the fma that forms kb has two constant operands and a DFMA takes at most one constant:
  // load both into registers once (opaque to the compiler, so it cannot re-materialise them)
  KdeRegs R;
  asm volatile("mov.b64 %0, %1;" : "=d"(R.log2e) : "d"(c_kde[0]));
  asm volatile("mov.b64 %0, %1;" : "=d"(R.magic) : "d"(C_MAGIC));
  for (;;) {
    u32 item = 0;
    if (lane == 0) item = (u32)atomicAdd(counter, 1ull);
    item = __shfl_sync(0xffffffffu, item, 0);
    if (item >= items) break;
    u32 tile = item_tile[item];
    u32 s = tile / tps, t = tile % tps;
    const SegDev& g = segs[s];
    u64 va = tile_range[2 * (u64)tile] + (u64)(item - tile_items[tile]) * KDE_CH;
    u64 ve = tile_range[2 * (u64)tile + 1];
    u32 len = (u32)min((u64)KDE_CH, ve - va);
    for (u32 i = lane; i < len; i += 32) sx[i] = __ull2double_rn(keys[va + i] & xmask);
    __syncwarp();
    const u32 slice = lane / KDE_TJ;
    u32 j = t * KDE_TJ + lane % KDE_TJ;
    double inv_h = g.inv_h;
    double gj = grid_pt(g.lo, g.hi, j < G ? j : G - 1, G);
    u64 acc = 0;
    u32 i = slice;
    const double* sSb = sS;
#if KDE_UNROLL > 4
    for (; i + (KDE_UNROLL - 1) * KDE_V < len; i += KDE_UNROLL * KDE_V) {
      u64 b[KDE_UNROLL];
#pragma unroll
      for (int q = 0; q < KDE_UNROLL; q++) b[q] = kde_qbits<GUARD>(gj, sx[i + q * KDE_V], inv_h, sSb, R);
#pragma unroll
      for (int q = 1; q < KDE_UNROLL; q++) b[0] += b[q];  // integer sums: order is irrelevant
      acc += b[0];
    }
#endif
    for (; i + 3 * KDE_V < len; i += 4 * KDE_V) {
      u64 b0 = kde_qbits<GUARD>(gj, sx[i], inv_h, sSb, R);
      u64 b1 = kde_qbits<GUARD>(gj, sx[i + KDE_V], inv_h, sSb, R);
      u64 b2 = kde_qbits<GUARD>(gj, sx[i + 2 * KDE_V], inv_h, sSb, R);
      u64 b3 = kde_qbits<GUARD>(gj, sx[i + 3 * KDE_V], inv_h, sSb, R);
      acc += (b0 + b1) + (b2 + b3);
    }
    for (; i < len; i += KDE_V) acc += kde_qbits<GUARD>(gj, sx[i], inv_h, sSb, R);
    // remove 2^52's bit pattern once per term this lane evaluated, then sum the value slices
    u32 nterm = len > slice ? (len - slice + KDE_V - 1) / KDE_V : 0;
    acc -= (u64)nterm * 0x4330000000000000ull;
#pragma unroll
    for (int o = KDE_TJ; o < 32; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (terms && lane == 0) {  // evaluated (lane, value) pairs of this item, wasted ones included
      u32 live = min((u32)KDE_TJ, G - t * KDE_TJ);
      atomicAdd(terms + 1, (unsigned long long)live * len);
    }
    if (j < G && slice == 0) {
      if (acc) {
        unsigned long long* d = (unsigned long long*)(D + 2 * ((u64)s * G + j));
        unsigned long long old = atomicAdd(d, (unsigned long long)acc);
        if (old + acc < old) atomicAdd(d + 1, 1ull);
      }
      if (terms) {  // values with |g - x| <= sqrt(74) h in this chunk (diagnostic work count)
        double wc = __dmul_rn(KDE_WC, g.h);
        double lo = __dsub_rn(gj, wc), hi = __dadd_rn(gj, wc);
        u32 l = 0, r = len;
        while (l < r) { u32 m = (l + r) >> 1; if (sx[m] < lo) l = m + 1; else r = m; }
        u32 a = l;
        r = len;
        while (l < r) { u32 m = (l + r) >> 1; if (sx[m] <= hi) l = m + 1; else r = m; }
        inwin += l - a;
      }
    }
    __syncwarp();
  }
  if (terms) {
    for (int o = 16; o > 0; o >>= 1) inwin += __shfl_down_sync(0xffffffffu, inwin, o);
    if (lane == 0 && inwin) atomicAdd(terms, (unsigned long long)inwin);
  }
}

size_t kde_item_bytes(u32 items) { return (size_t)items * 4 + 16; }

void launch_kde(const SegDev* segs, u32 nseg, u32 G, const u64* keys, u64 xmask,
                const u64* tile_range, const u32* tile_items, u32* item_tile, u32 items, u64* D,
                unsigned long long* work_counter, unsigned long long* terms, bool guard,
                cudaStream_t s) {
  if (items == 0) return;
  u32 tps = div_up(G, KDE_TJ);
  u32 ntiles = nseg * tps;
  // `items` is a host-side upper bound: grids are sized by it, the kernels stop at the
  // device-side count tile_items[ntiles]
  SV_LAUNCH(k_kde_items, min(div_up(items, 256), 4096u), 256, 0, s)(tile_items, ntiles, item_tile);
  auto kern = guard ? k_kde<true> : k_kde<false>;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, KDE_SMEM_BYTES);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 32 * KDE_WARPS, KDE_SMEM_BYTES);
  if (per_sm < 1) per_sm = 1;
  u32 grid = (u32)sv_num_sms() * (u32)per_sm;
  u32 need = div_up(items, KDE_WARPS);
  if (grid > need) grid = need;
  cudaMemsetAsync(work_counter, 0, 8, s);
  SV_LAUNCH(kern, grid, 32 * KDE_WARPS, KDE_SMEM_BYTES, s)(segs, G, tps, keys, xmask, tile_range,
                                                           tile_items, item_tile, ntiles, D,
                                                           work_counter, terms);
}
