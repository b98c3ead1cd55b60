// sort.cu -- Tier-3 key compaction, LSD radix sort of 64-bit packed keys, exclusive scans and
// the u128 prefix sums of x and x^2 over the sorted Tier-3 values.
//
// The north_star path sorts (kernel, instruction count) to group each high-CoV kernel's
// invocations by value (the KDE windows and the part moments need them contiguous).  Only
// Tier-3 invocations are sorted (A-series reading "sort only Tier-3 keys"); the
// key is (t3rank << bx) + x with bx = bitlen(max x), so only ceil(bits / 8) digit passes run,
// and passes whose 8 bits are constant over all keys (found by one OR-reduction of key ^ key0)
// are skipped.
//
// Radix pass = reduce-then-scan: per-tile digit histograms (warp-aggregated with match.any),
// one exclusive scan over the digit-major [digit][tile] matrix, then a scatter that ranks keys
// stably inside the tile (match.any per 32-key round), stages them in shared memory in tile
// order and writes runs of equal digits coalesced.
#include "kernels.cuh"

#define RS_THREADS 256
#define RS_IPT 16
#define RS_TILE (RS_THREADS * RS_IPT)
#define RS_WARPS (RS_THREADS / 32)

// ------------------------------------------------------------------------------------------
// block-wide exclusive scan helpers
// ------------------------------------------------------------------------------------------
template <typename T>
__device__ __forceinline__ T sv_zero() { return T(0); }
template <typename T>
__device__ __forceinline__ T warp_incl_scan(T v) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T n = __shfl_up_sync(0xffffffffu, v, o);
    if ((int)lane_id() >= o) v += n;
  }
  return v;
}

// returns exclusive prefix of v over the block; *total receives the block sum
template <typename T, int NT>
__device__ __forceinline__ T block_excl_scan(T v, T* total) {
  __shared__ T s_w[NT / 32];
  T inc = warp_incl_scan(v);
  u32 w = threadIdx.x >> 5;
  if (lane_id() == 31) s_w[w] = inc;
  __syncthreads();
  if (w == 0) {
    T t = lane_id() < NT / 32 ? s_w[lane_id()] : sv_zero<T>();
    T ti = warp_incl_scan(t);
    if (lane_id() < NT / 32) s_w[lane_id()] = ti - t;
    if (lane_id() == NT / 32 - 1) *total = ti;
  }
  __syncthreads();
  T r = s_w[w] + inc - v;
  __syncthreads();
  return r;
}

// ------------------------------------------------------------------------------------------
// u32 exclusive scan (3 phases), used for radix offsets and KDE work-item counts
// ------------------------------------------------------------------------------------------
#define SC_THREADS 1024
#define SC_IPT 4
#define SC_TILE (SC_THREADS * SC_IPT)

__global__ void __launch_bounds__(SC_THREADS) k_scan_reduce(const u32* in, u64 n, u32* bsum) {
  u64 base = (u64)blockIdx.x * SC_TILE;
  u32 s = 0;
#pragma unroll
  for (int j = 0; j < SC_IPT; j++) {
    u64 i = base + (u64)j * SC_THREADS + threadIdx.x;
    if (i < n) s += in[i];
  }
  __shared__ u32 tot;
  block_excl_scan<u32, SC_THREADS>(s, &tot);
  if (threadIdx.x == 0) bsum[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(SC_THREADS) k_scan_blocks(u32* bsum, u32 nb, u32* total) {
  __shared__ u32 carry_s;
  if (threadIdx.x == 0) carry_s = 0;
  __syncthreads();
  for (u32 b0 = 0; b0 < nb; b0 += SC_THREADS) {
    u32 i = b0 + threadIdx.x;
    u32 v = i < nb ? bsum[i] : 0;
    __shared__ u32 tot;
    u32 ex = block_excl_scan<u32, SC_THREADS>(v, &tot);
    u32 c = carry_s;
    if (i < nb) bsum[i] = c + ex;
    __syncthreads();
    if (threadIdx.x == 0) carry_s = c + tot;
    __syncthreads();
  }
  if (threadIdx.x == 0 && total) *total = carry_s;
}

__global__ void __launch_bounds__(SC_THREADS) k_scan_apply(const u32* in, u64 n, const u32* bsum,
                                                           u32* out) {
  u64 base = (u64)blockIdx.x * SC_TILE + (u64)threadIdx.x * SC_IPT;
  u32 v[SC_IPT];
  u32 s = 0;
#pragma unroll
  for (int j = 0; j < SC_IPT; j++) {
    v[j] = base + j < n ? in[base + j] : 0;
    s += v[j];
  }
  __shared__ u32 tot;
  u32 ex = block_excl_scan<u32, SC_THREADS>(s, &tot) + bsum[blockIdx.x];
#pragma unroll
  for (int j = 0; j < SC_IPT; j++) {
    if (base + j < n) out[base + j] = ex;
    ex += v[j];
  }
}

size_t scan_u32_temp_bytes(u64 n) { return ((n + SC_TILE - 1) / SC_TILE + 2) * sizeof(u32); }

// exclusive scan in -> out (may alias); total (device pointer, nullable) receives the sum
void scan_u32(const u32* in, u32* out, u64 n, void* temp, u32* total, cudaStream_t s) {
  u32 nb = div_up(n ? n : 1, SC_TILE);
  u32* bsum = (u32*)temp;
  SV_LAUNCH(k_scan_reduce, nb, SC_THREADS, 0, s)(in, n, bsum);
  SV_LAUNCH(k_scan_blocks, 1, SC_THREADS, 0, s)(bsum, nb, total);
  SV_LAUNCH(k_scan_apply, nb, SC_THREADS, 0, s)(in, n, bsum, out);
}

// ------------------------------------------------------------------------------------------
// Tier-3 compaction: one global atomic per 4096-row tile; order inside a tile is preserved
// (the order does not matter: the keys are sorted next)
// ------------------------------------------------------------------------------------------
#define CP_THREADS 512
#define CP_IPT 8
__global__ void __launch_bounds__(CP_THREADS)
k_t3_compact(const u32* __restrict__ kid, const u64* __restrict__ x, u64 n,
             const u32* __restrict__ t3rank, u32 bx, u64* __restrict__ keys,
             unsigned long long* counter) {
  const u64 tile = (u64)CP_THREADS * CP_IPT;
  for (u64 base = (u64)blockIdx.x * tile; base < n; base += (u64)gridDim.x * tile) {
    u64 key[CP_IPT];
    u32 cnt = 0;
#pragma unroll
    for (int j = 0; j < CP_IPT; j++) {
      u64 i = base + (u64)j * CP_THREADS + threadIdx.x;
      key[j] = ~0ull;
      if (i < n) {
        u32 r = t3rank[__ldcs(kid + i)];
        if (r != 0xFFFFFFFFu) { key[j] = ((u64)r << bx) + __ldcs(x + i); cnt++; }
      }
    }
    __shared__ u32 tot;
    __shared__ unsigned long long gbase;
    u32 ex = block_excl_scan<u32, CP_THREADS>(cnt, &tot);
    if (threadIdx.x == 0) gbase = tot ? atomicAdd(counter, (unsigned long long)tot) : 0ull;
    __syncthreads();
    u64 o = gbase + ex;
#pragma unroll
    for (int j = 0; j < CP_IPT; j++)
      if (key[j] != ~0ull) keys[o++] = key[j];
    __syncthreads();
  }
}

void launch_t3_compact(const u32* kid, const u64* x, u64 n, const u32* t3rank, u32 bx,
                       u64* keys_out, unsigned long long* counter, cudaStream_t s) {
  if (n == 0) return;
  u64 tiles = (n + (u64)CP_THREADS * CP_IPT - 1) / ((u64)CP_THREADS * CP_IPT);
  u64 grid = tiles < (u64)sv_num_sms() * 4 ? tiles : (u64)sv_num_sms() * 4;
  SV_LAUNCH(k_t3_compact, (unsigned)grid, CP_THREADS, 0, s)(kid, x, n, t3rank, bx, keys_out, counter);
}

// ------------------------------------------------------------------------------------------
// radix sort
// ------------------------------------------------------------------------------------------
__global__ void k_or_diff(const u64* keys, u64 n, u64* mask) {
  u64 k0 = keys[0];
  u64 m = 0;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x)
    m |= keys[i] ^ k0;
  for (int o = 16; o > 0; o >>= 1) m |= __shfl_down_sync(0xffffffffu, m, o);
  if (lane_id() == 0 && m) atomicOr((unsigned long long*)mask, m);
}

__global__ void __launch_bounds__(RS_THREADS)
k_rs_hist(const u64* __restrict__ keys, u64 n, int shift, u32 ntiles, u32* __restrict__ hist) {
  __shared__ u32 s_h[RS_WARPS][256];
  for (int i = threadIdx.x; i < RS_WARPS * 256; i += RS_THREADS) (&s_h[0][0])[i] = 0;
  __syncthreads();
  u32 w = threadIdx.x >> 5;
  u64 base = (u64)blockIdx.x * RS_TILE + (u64)w * (RS_TILE / RS_WARPS);
  u32 dig[RS_IPT];  // all loads of the tile in flight before any ranking
#pragma unroll
  for (int r = 0; r < RS_IPT; r++) {
    u64 i = base + (u64)r * 32 + lane_id();
    dig[r] = i < n ? (u32)(__ldcs(keys + i) >> shift) & 255u : 256u;
  }
#pragma unroll
  for (int r = 0; r < RS_IPT; r++) {
    u32 d = dig[r];
    u32 peers = __match_any_sync(0xffffffffu, d);
    if (d < 256u && lane_id() == (u32)(__ffs(peers) - 1)) s_h[w][d] += __popc(peers);
    __syncwarp();
  }
  __syncthreads();
  u32 d = threadIdx.x;  // RS_THREADS == 256 digits
  u32 s = 0;
#pragma unroll
  for (int j = 0; j < RS_WARPS; j++) s += s_h[j][d];
  hist[(u64)d * ntiles + blockIdx.x] = s;
}

__global__ void __launch_bounds__(RS_THREADS)
k_rs_scatter(const u64* __restrict__ kin, const u32* __restrict__ vin, u64 n, int shift,
             u32 ntiles, const u32* __restrict__ off, u64* __restrict__ kout,
             u32* __restrict__ vout) {
  extern __shared__ __align__(16) unsigned char smem[];
  u64* s_k = (u64*)smem;                        // [RS_TILE]
  u32* s_v = (u32*)(s_k + RS_TILE);             // [RS_TILE] (if values)
  __shared__ u32 s_wh[RS_WARPS][256];           // per-warp digit counts -> warp offsets
  __shared__ u32 s_td[256];                     // tile-local digit offsets
  __shared__ u32 s_go[256];                     // global digit offsets of this tile
  for (int i = threadIdx.x; i < RS_WARPS * 256; i += RS_THREADS) (&s_wh[0][0])[i] = 0;
  __syncthreads();
  u32 w = threadIdx.x >> 5;
  u64 base = (u64)blockIdx.x * RS_TILE + (u64)w * (RS_TILE / RS_WARPS);
  u64 key[RS_IPT];
  u32 val[RS_IPT];
  u32 rank[RS_IPT];
#pragma unroll
  for (int r = 0; r < RS_IPT; r++) {  // all loads of the tile in flight before any ranking
    u64 i = base + (u64)r * 32 + lane_id();
    bool ok = i < n;
    key[r] = ok ? __ldcs(kin + i) : 0;
    val[r] = (ok && vin) ? __ldcs(vin + i) : 0;
  }
#pragma unroll
  for (int r = 0; r < RS_IPT; r++) {
    u64 i = base + (u64)r * 32 + lane_id();
    bool ok = i < n;
    u32 d = ok ? (u32)(key[r] >> shift) & 255u : 256u;
    u32 peers = __match_any_sync(0xffffffffu, d);
    u32 lt = peers & ((1u << lane_id()) - 1u);
    u32 cur = d < 256u ? s_wh[w][d] : 0;
    rank[r] = cur + __popc(lt);
    __syncwarp();
    if (d < 256u && lt == 0) s_wh[w][d] = cur + __popc(peers);
    __syncwarp();
  }
  __syncthreads();
  {  // thread d: exclusive over warps, then exclusive over digits
    u32 d = threadIdx.x;
    u32 run = 0;
#pragma unroll
    for (int j = 0; j < RS_WARPS; j++) { u32 c = s_wh[j][d]; s_wh[j][d] = run; run += c; }
    __shared__ u32 tot;
    u32 ex = block_excl_scan<u32, RS_THREADS>(run, &tot);
    s_td[d] = ex;
    s_go[d] = off[(u64)d * ntiles + blockIdx.x];
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < RS_IPT; r++) {
    u64 i = base + (u64)r * 32 + lane_id();
    if (i < n) {
      u32 d = (u32)(key[r] >> shift) & 255u;
      u32 p = s_td[d] + s_wh[w][d] + rank[r];
      s_k[p] = key[r];
      if (vin) s_v[p] = val[r];
    }
  }
  __syncthreads();
  u64 tile_n = n - (u64)blockIdx.x * RS_TILE;
  if (tile_n > RS_TILE) tile_n = RS_TILE;
  for (u32 j = threadIdx.x; j < tile_n; j += RS_THREADS) {
    u64 k = s_k[j];
    u32 d = (u32)(k >> shift) & 255u;
    u64 o = (u64)s_go[d] + (j - s_td[d]);
    kout[o] = k;
    if (vin) vout[o] = s_v[j];
  }
}

size_t radix_sort_temp_bytes(u64 n, bool with_vals) {
  u64 ntiles = (n + RS_TILE - 1) / RS_TILE;
  size_t b = 0;
  b += ((n * 8 + 255) / 256) * 256;                       // alt keys
  if (with_vals) b += ((n * 4 + 255) / 256) * 256;        // alt vals
  b += ((256 * ntiles * 4 + 255) / 256) * 256;            // histogram / offsets
  b += ((scan_u32_temp_bytes(256 * ntiles) + 255) / 256) * 256;
  b += 256;                                               // diff mask
  return b;
}

int radix_sort(u64* keys, u32* vals, u64 n, int nbits, void* temp, cudaStream_t s, int* passes) {
  if (passes) *passes = 0;
  if (n <= 1 || nbits <= 0) return SIEVE_OK;
  u64 ntiles = (n + RS_TILE - 1) / RS_TILE;
  char* t = (char*)temp;
  u64* kalt = (u64*)t; t += ((n * 8 + 255) / 256) * 256;
  u32* valt = nullptr;
  if (vals) { valt = (u32*)t; t += ((n * 4 + 255) / 256) * 256; }
  u32* hist = (u32*)t; t += ((256 * ntiles * 4 + 255) / 256) * 256;
  void* stemp = t; t += ((scan_u32_temp_bytes(256 * ntiles) + 255) / 256) * 256;
  u64* dmask = (u64*)t;
  SV_CUDA(cudaMemsetAsync(dmask, 0, 8, s));
  SV_LAUNCH(k_or_diff, sv_num_sms() * 2, 256, 0, s)(keys, n, dmask);
  u64 mask = 0;
  SV_CUDA(cudaMemcpyAsync(&mask, dmask, 8, cudaMemcpyDeviceToHost, s));
  SV_CUDA(cudaStreamSynchronize(s));
  size_t smem = (size_t)RS_TILE * (8 + 4);
  SV_CUDA(cudaFuncSetAttribute(k_rs_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  u64* kin = keys; u32* vin = vals; u64* kout = kalt; u32* vout = valt;
  for (int shift = 0; shift < nbits; shift += 8) {
    if (((mask >> shift) & 255u) == 0) continue;   // constant digit: the pass is the identity
    SV_LAUNCH(k_rs_hist, (unsigned)ntiles, RS_THREADS, 0, s)(kin, n, shift, (u32)ntiles, hist);
    scan_u32(hist, hist, 256 * ntiles, stemp, nullptr, s);
    SV_LAUNCH(k_rs_scatter, (unsigned)ntiles, RS_THREADS, smem, s)(kin, vin, n, shift, (u32)ntiles, hist,
                                                            kout, vout);
    u64* tk = kin; kin = kout; kout = tk;
    u32* tv = vin; vin = vout; vout = tv;
    if (passes) (*passes)++;
  }
  if (kin != keys) {
    SV_CUDA(cudaMemcpyAsync(keys, kin, n * 8, cudaMemcpyDeviceToDevice, s));
    if (vals) SV_CUDA(cudaMemcpyAsync(vals, vin, n * 4, cudaMemcpyDeviceToDevice, s));
  }
  SV_CUDA(cudaGetLastError());
  return SIEVE_OK;
}

// ------------------------------------------------------------------------------------------
// u128 prefix sums of x and x^2 over the sorted keys (x = key & xmask)
// ------------------------------------------------------------------------------------------
// POD u128 / pair types (no constructors: they live in __shared__ memory)
struct U128 { u64 lo, hi; };
struct Pair128 { U128 a, b; };
__device__ __forceinline__ U128 add128v(U128 x, U128 y) {
  U128 r; r.lo = x.lo + y.lo; r.hi = x.hi + y.hi + (r.lo < x.lo ? 1ull : 0ull); return r;
}
__device__ __forceinline__ U128 sub128v(U128 x, U128 y) {
  U128 r; r.lo = x.lo - y.lo; r.hi = x.hi - y.hi - (x.lo < y.lo ? 1ull : 0ull); return r;
}
__device__ __forceinline__ Pair128 operator+(const Pair128& x, const Pair128& y) {
  Pair128 r; r.a = add128v(x.a, y.a); r.b = add128v(x.b, y.b); return r;
}
__device__ __forceinline__ Pair128& operator+=(Pair128& x, const Pair128& y) { x = x + y; return x; }
__device__ __forceinline__ Pair128 operator-(const Pair128& x, const Pair128& y) {
  Pair128 r; r.a = sub128v(x.a, y.a); r.b = sub128v(x.b, y.b); return r;
}
__device__ __forceinline__ Pair128 pzero() { Pair128 r; r.a.lo = r.a.hi = r.b.lo = r.b.hi = 0; return r; }
template <>
__device__ __forceinline__ Pair128 sv_zero<Pair128>() { return pzero(); }
template <>
__device__ __forceinline__ Pair128 warp_incl_scan<Pair128>(Pair128 v) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    Pair128 n;
    n.a.lo = __shfl_up_sync(0xffffffffu, v.a.lo, o); n.a.hi = __shfl_up_sync(0xffffffffu, v.a.hi, o);
    n.b.lo = __shfl_up_sync(0xffffffffu, v.b.lo, o); n.b.hi = __shfl_up_sync(0xffffffffu, v.b.hi, o);
    if ((int)lane_id() >= o) v += n;
  }
  return v;
}

#define PX_THREADS 512
#define PX_IPT 8
#define PX_TILE (PX_THREADS * PX_IPT)

__device__ __forceinline__ Pair128 px_val(u64 key, u64 xmask) {
  u64 x = key & xmask;
  Pair128 r; r.a.lo = x; r.a.hi = 0; r.b.lo = x * x; r.b.hi = __umul64hi(x, x); return r;
}

__global__ void __launch_bounds__(PX_THREADS)
k_px_reduce(const u64* keys, u64 n, u64 xmask, Pair128* bsum) {
  u64 base = (u64)blockIdx.x * PX_TILE + (u64)threadIdx.x * PX_IPT;
  Pair128 s = pzero();
#pragma unroll
  for (int j = 0; j < PX_IPT; j++)
    if (base + j < n) s += px_val(keys[base + j], xmask);
  __shared__ Pair128 tot;
  block_excl_scan<Pair128, PX_THREADS>(s, &tot);
  if (threadIdx.x == 0) bsum[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(PX_THREADS) k_px_blocks(Pair128* bsum, u32 nb) {
  __shared__ Pair128 carry_s;
  if (threadIdx.x == 0) carry_s = pzero();
  __syncthreads();
  for (u32 b0 = 0; b0 < nb; b0 += PX_THREADS) {
    u32 i = b0 + threadIdx.x;
    Pair128 v = i < nb ? bsum[i] : pzero();
    __shared__ Pair128 tot;
    Pair128 ex = block_excl_scan<Pair128, PX_THREADS>(v, &tot);
    Pair128 c = carry_s;
    if (i < nb) bsum[i] = c + ex;
    __syncthreads();
    if (threadIdx.x == 0) carry_s = c + tot;
    __syncthreads();
  }
}

__global__ void __launch_bounds__(PX_THREADS)
k_px_apply(const u64* keys, u64 n, u64 xmask, const Pair128* bsum, u64* P1, u64* P2) {
  u64 base = (u64)blockIdx.x * PX_TILE + (u64)threadIdx.x * PX_IPT;
  Pair128 v[PX_IPT];
  Pair128 s = pzero();
#pragma unroll
  for (int j = 0; j < PX_IPT; j++) {
    v[j] = base + j < n ? px_val(keys[base + j], xmask) : pzero();
    s += v[j];
  }
  __shared__ Pair128 tot;
  Pair128 ex = block_excl_scan<Pair128, PX_THREADS>(s, &tot) + bsum[blockIdx.x];
#pragma unroll
  for (int j = 0; j < PX_IPT; j++) {
    if (base + j <= n) {
      P1[2 * (base + j)] = ex.a.lo; P1[2 * (base + j) + 1] = ex.a.hi;
      P2[2 * (base + j)] = ex.b.lo; P2[2 * (base + j) + 1] = ex.b.hi;
    }
    ex += v[j];
  }
}

size_t prefix128_temp_bytes(u64 n) { return ((n + PX_TILE) / PX_TILE + 2) * sizeof(Pair128); }

void launch_prefix128(const u64* keys, u64 n, u64 xmask, u64* P1, u64* P2, void* temp,
                      cudaStream_t s) {
  // n+1 outputs: cover index n with one extra element slot
  u32 nb = div_up(n + 1, PX_TILE);
  Pair128* bsum = (Pair128*)temp;
  SV_LAUNCH(k_px_reduce, nb, PX_THREADS, 0, s)(keys, n, xmask, bsum);
  SV_LAUNCH(k_px_blocks, 1, PX_THREADS, 0, s)(bsum, nb);
  SV_LAUNCH(k_px_apply, nb, PX_THREADS, 0, s)(keys, n, xmask, bsum, P1, P2);
}
