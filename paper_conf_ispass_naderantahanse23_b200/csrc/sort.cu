// sort.cu -- Tier-3 key compaction, LSD radix sort of 64-bit packed keys and exclusive scans.
//
// The compaction gathers the Tier-3 invocations as keys (t3rank << bx) + x (bx = bitlen(max x)).
// The radix sort orders them per refinement round by (segment, grid cell) (bucket.cu: the cell
// keys' low bits), and also the (stratum, CTA) entries of pass B, the name hashes of the CSV
// ingest and the Tier-3 keys of the exact min-strata DP.  It runs one onesweep pass per 8-bit
// digit of the key bits it is asked to sort (see below): digit histograms and bases are computed
// on the device, with no host read-back.
#include <algorithm>

#include "kernels.cuh"

#ifndef RS_THREADS
#define RS_THREADS 256
#endif
#ifndef RS_IPT
#define RS_IPT 12     // A/B on C4: 12 keys x 3 blocks/SM beat 16 x 2 by ~3% (8 x 4, 20 x 2 no better)
#endif
#ifndef RS_MINB
#define RS_MINB 3
#endif
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
  pdl_begin();
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
  pdl_begin();
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
  pdl_begin();
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

// small scans (up to SC_SMALL tiles: the per-round KDE tile and part counts) in ONE block that
// walks the tiles with a carry: one launch instead of three (the host launch cost between
// synchronisations is GPU idle time)
#define SC_SMALL 4
__global__ void __launch_bounds__(SC_THREADS) k_scan_single(const u32* in, u64 n, u32* out, u32* total) {
  pdl_begin();
  __shared__ u32 carry_s;
  if (threadIdx.x == 0) carry_s = 0;
  __syncthreads();
  for (u64 t0 = 0; t0 < n; t0 += SC_TILE) {
    const u64 base = t0 + (u64)threadIdx.x * SC_IPT;
    u32 v[SC_IPT];
    u32 sum = 0;
#pragma unroll
    for (int j = 0; j < SC_IPT; j++) {
      v[j] = base + j < n ? in[base + j] : 0;
      sum += v[j];
    }
    __shared__ u32 tot;
    u32 ex = block_excl_scan<u32, SC_THREADS>(sum, &tot) + carry_s;
#pragma unroll
    for (int j = 0; j < SC_IPT; j++) {
      if (base + j < n) out[base + j] = ex;
      ex += v[j];
    }
    __syncthreads();
    if (threadIdx.x == 0) carry_s += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0 && total) *total = carry_s;
}

size_t scan_u32_temp_bytes(u64 n) { return ((n + SC_TILE - 1) / SC_TILE + 2) * sizeof(u32); }

// look-back status words: GPU-scope relaxed accesses (served by L2; volatile would be
// system scope).  Each word is written whole, so a reader sees either 0 or a complete value.
__device__ __forceinline__ u64 ld_volatile_u64(const u64* p) {
  u64 v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_volatile_u64(u64* p, u64 v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// ------------------------------------------------------------------------------------------
// single-pass scan (one launch instead of three): tiles taken from a ticket counter, decoupled
// look-back over 64-bit status words (2 flag bits + 62-bit sum).  The status words, the ticket
// and the done counter live in a per-context persistent buffer that starts zeroed and is
// re-zeroed by the last tile to finish, so no memset is launched.
// ------------------------------------------------------------------------------------------
#define SP_FLAG_AGG (1ull << 62)
#define SP_FLAG_PRE (2ull << 62)
#define SP_VAL ((1ull << 62) - 1)
static thread_local u64* tl_scan_state = nullptr;   // [SCAN_SP_MAX_TILES + 2] on the device
void scan_set_state(u64* state) { tl_scan_state = state; }

__global__ void __launch_bounds__(SC_THREADS) k_scan_sp(const u32* in, u32* out, u64 n, u32 ntiles, u64* st,
                                                        u32* total) {
  pdl_begin();
  __shared__ u32 s_tile;
  __shared__ u64 s_excl;
  __shared__ bool s_last;
  unsigned int* ticket = (unsigned int*)(st + SCAN_SP_MAX_TILES);
  unsigned int* done = ticket + 1;
  if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
  __syncthreads();
  const u32 tile = s_tile;
  const u64 base = (u64)tile * SC_TILE + (u64)threadIdx.x * SC_IPT;
  u32 v[SC_IPT];
  u32 sum = 0;
#pragma unroll
  for (int j = 0; j < SC_IPT; j++) {
    v[j] = base + j < n ? in[base + j] : 0;
    sum += v[j];
  }
  __shared__ u32 tot;
  u32 ex = block_excl_scan<u32, SC_THREADS>(sum, &tot);
  if (threadIdx.x == 0) {
    u64 excl = 0;
    if (tile == 0) {
      st_volatile_u64(st, SP_FLAG_PRE | tot);
    } else {
      st_volatile_u64(st + tile, SP_FLAG_AGG | tot);
      for (int j = (int)tile - 1; j >= 0; j--) {
        u64 w;
        do { w = ld_volatile_u64(st + j); } while ((w >> 62) == 0);
        excl += w & SP_VAL;
        if (w & SP_FLAG_PRE) break;
      }
      st_volatile_u64(st + tile, SP_FLAG_PRE | (excl + tot));
    }
    s_excl = excl;
    if (tile == ntiles - 1 && total) *total = (u32)(excl + tot);
  }
  __syncthreads();
  u32 run = (u32)s_excl + ex;
#pragma unroll
  for (int j = 0; j < SC_IPT; j++) {
    if (base + j < n) out[base + j] = run;
    run += v[j];
  }
  // the last tile to finish (every look-back is over by then) re-zeroes the state
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(done, 1u) == ntiles - 1;
  }
  __syncthreads();
  if (s_last) {
    for (u32 j = threadIdx.x; j < ntiles; j += SC_THREADS) st[j] = 0;
    if (threadIdx.x == 0) { *ticket = 0; *done = 0; }
  }
}

// exclusive scan in -> out (may alias); total (device pointer, nullable) receives the sum
void scan_u32(const u32* in, u32* out, u64 n, void* temp, u32* total, cudaStream_t s) {
  u32 nb = div_up(n ? n : 1, SC_TILE);
  if (nb <= SC_SMALL) {
    SV_LAUNCH(k_scan_single, 1, SC_THREADS, 0, s)(in, n, out, total);
    return;
  }
  if (tl_scan_state && nb <= SCAN_SP_MAX_TILES) {
    SV_LAUNCH(k_scan_sp, nb, SC_THREADS, 0, s)(in, out, n, nb, tl_scan_state, total);
    return;
  }
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
  pdl_begin();
  const u64 tile = (u64)CP_THREADS * CP_IPT;
  for (u64 base = (u64)blockIdx.x * tile; base < n; base += (u64)gridDim.x * tile) {
    u64 key[CP_IPT];
    u32 kk[CP_IPT];
    u32 cnt = 0;
#pragma unroll
    for (int j = 0; j < CP_IPT; j++) {  // all independent loads first
      u64 i = base + (u64)j * CP_THREADS + threadIdx.x;
      bool ok = i < n;
      kk[j] = ok ? __ldcs(kid + i) : 0u;
      key[j] = ok ? __ldcs(x + i) : ~0ull;
    }
#pragma unroll
    for (int j = 0; j < CP_IPT; j++) {
      u64 i = base + (u64)j * CP_THREADS + threadIdx.x;
      u32 r = i < n ? __ldg(t3rank + kk[j]) : 0xFFFFFFFFu;
      if (r != 0xFFFFFFFFu) { key[j] = ((u64)r << bx) + key[j]; cnt++; }
      else key[j] = ~0ull;
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
// ------------------------------------------------------------------------------------------
// Onesweep (single-pass per digit) radix sort.  One upfront kernel reads the keys once and
// builds the global 256-bin histogram of EVERY digit position; the host reads them back once
// (skipping digits whose histogram has a single non-empty bin: that pass is the identity) and
// scans them into global digit bases.  Each digit pass is then ONE kernel: a block takes the
// next tile from an atomic counter (so predecessors are always resident), ranks its keys
// stably (match.any per 32-key round), publishes its per-digit counts, and obtains its
// exclusive per-digit prefix by decoupled look-back over the predecessors' published
// aggregates / inclusive prefixes (64-bit status words: 2 flag bits + 62-bit count), then
// scatters through shared memory in runs of equal digits.  16 B of HBM traffic per key per
// pass (read + write), versus 24 B for reduce-then-scan.
// ------------------------------------------------------------------------------------------
#define OS_FLAG_AGG (1ull << 62)
#define OS_FLAG_PREFIX (2ull << 62)
#define OS_VALUE_MASK ((1ull << 62) - 1)
#define OS_MAX_PASSES 8
#ifndef OS_LB
#define OS_LB 4   // predecessors read per look-back step
#endif

__global__ void __launch_bounds__(RS_THREADS)
k_os_hist(const u64* __restrict__ keys, u64 n, int npass, u64 kmask, u32* __restrict__ ghist) {
  pdl_begin();
  extern __shared__ u32 s_hist[];  // [RS_WARPS/2][npass][256] (pairs of warps share a table)
  const int tables = RS_WARPS / 2;
  for (int i = threadIdx.x; i < tables * npass * 256; i += RS_THREADS) s_hist[i] = 0;
  __syncthreads();
  u32* mine = s_hist + (threadIdx.x >> 6) * npass * 256;
  for (u64 i = (u64)blockIdx.x * RS_THREADS + threadIdx.x; i < n; i += (u64)gridDim.x * RS_THREADS) {
    u64 k = __ldcs(keys + i) & kmask;
    for (int p = 0; p < npass; p++) atomicAdd(&mine[p * 256 + ((k >> (8 * p)) & 255u)], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < npass * 256; i += RS_THREADS) {
    u32 s = 0;
    for (int t = 0; t < tables; t++) s += s_hist[t * npass * 256 + i];
    if (s) atomicAdd(&ghist[i], s);
  }
}

template <bool V>  // V: a u32 payload travels with each key
__global__ void __launch_bounds__(RS_THREADS, RS_MINB)
k_os_pass(const u64* __restrict__ kin, const u32* __restrict__ vin, u64 n, int shift, u32 dmask,
          const u32* __restrict__ gbase, u64* status, u32* tile_counter, u64* __restrict__ kout,
          u32* __restrict__ vout) {
  pdl_begin();
  extern __shared__ __align__(16) unsigned char smem[];
  const int dbits = __popc(dmask);
  u64* s_k = (u64*)smem;                        // [RS_TILE]
  u32* s_v = (u32*)(s_k + RS_TILE);             // [RS_TILE] (if values)
  __shared__ u32 s_wh[RS_WARPS][256];           // per-warp digit counts -> warp offsets
  __shared__ u32 s_td[256];                     // tile-local digit offsets
  __shared__ u64 s_go[256];                     // global digit offsets of this tile
  __shared__ u32 s_tile;
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_counter, 1u);
  for (int i = threadIdx.x; i < RS_WARPS * 256; i += RS_THREADS) (&s_wh[0][0])[i] = 0;
  __syncthreads();
  const u32 tile = s_tile;
  u32 w = threadIdx.x >> 5;
  u64 base = (u64)tile * RS_TILE + (u64)w * (RS_TILE / RS_WARPS);
  u64 key[RS_IPT];
  u32 val[RS_IPT];
  u32 rank[RS_IPT];
#pragma unroll
  for (int r = 0; r < RS_IPT; r++) {  // all loads of the tile in flight before any ranking
    u64 i = base + (u64)r * 32 + lane_id();
    bool ok = i < n;
    key[r] = ok ? __ldcs(kin + i) : 0;
    if (V) val[r] = ok ? __ldcs(vin + i) : 0;
  }
#pragma unroll
  for (int r = 0; r < RS_IPT; r++) {
    u64 i = base + (u64)r * 32 + lane_id();
    bool ok = i < n;
    u32 d = ok ? (u32)(key[r] >> shift) & dmask : 256u;
    // lanes with the same digit: 8 ballots (one per digit bit) plus validity, ANDed -- cheaper
    // than MATCH.ANY, which serialises in the MIO pipe
    u32 peers = __ballot_sync(0xffffffffu, ok);
    if (!ok) peers = ~peers;
#pragma unroll
    for (int b = 0; b < 8; b++) {
      if (b >= dbits) break;  // narrow last digit: fewer ballots (uniform branch)
      u32 m = __ballot_sync(0xffffffffu, (d >> b) & 1u);
      peers &= ((d >> b) & 1u) ? m : ~m;
    }
    u32 lt = peers & ((1u << lane_id()) - 1u);
    u32 cur = d < 256u ? s_wh[w][d] : 0;
    rank[r] = cur + __popc(lt);
    __syncwarp();
    if (d < 256u && lt == 0) s_wh[w][d] = cur + __popc(peers);
    __syncwarp();
  }
  __syncthreads();
  {  // thread d: warp offsets, tile count, publish, look back, tile-local digit offsets
    u32 d = threadIdx.x;
    u32 run = 0;
#pragma unroll
    for (int j = 0; j < RS_WARPS; j++) { u32 c = s_wh[j][d]; s_wh[j][d] = run; run += c; }
    u64* my = status + (u64)tile * 256 + d;
    u64 excl = 0;
    if (tile == 0) {
      st_volatile_u64(my, OS_FLAG_PREFIX | run);
    } else {
      st_volatile_u64(my, OS_FLAG_AGG | run);
      // look back OS_LB predecessors at a time: their status loads are in flight together
      // (each is an L2 round trip, possibly to the other die)
      bool done = false;
      for (int j0 = (int)tile - 1; !done; j0 -= OS_LB) {
        u64 v[OS_LB];
#pragma unroll
        for (int q = 0; q < OS_LB; q++)
          v[q] = j0 - q >= 0 ? ld_volatile_u64(status + (u64)(j0 - q) * 256 + d) : OS_FLAG_PREFIX;
#pragma unroll
        for (int q = 0; q < OS_LB; q++) {
          if (done) break;
          while ((v[q] >> 62) == 0) v[q] = ld_volatile_u64(status + (u64)(j0 - q) * 256 + d);
          excl += v[q] & OS_VALUE_MASK;
          if (v[q] & OS_FLAG_PREFIX) done = true;
        }
      }
      st_volatile_u64(my, OS_FLAG_PREFIX | (excl + run));
    }
    __shared__ u32 tot;
    u32 ex = block_excl_scan<u32, RS_THREADS>(run, &tot);
    s_td[d] = ex;
    s_go[d] = (u64)gbase[d] + excl;
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < RS_IPT; r++) {
    u64 i = base + (u64)r * 32 + lane_id();
    if (i < n) {
      u32 d = (u32)(key[r] >> shift) & dmask;
      u32 p = s_td[d] + s_wh[w][d] + rank[r];
      s_k[p] = key[r];
      if (V) s_v[p] = val[r];
    }
  }
  __syncthreads();
  u64 tile_n = n - (u64)tile * RS_TILE;
  if (tile_n > RS_TILE) tile_n = RS_TILE;
  for (u32 j = threadIdx.x; j < tile_n; j += RS_THREADS) {
    u64 k = s_k[j];
    u32 d = (u32)(k >> shift) & dmask;
    u64 o = s_go[d] + (j - s_td[d]);
    kout[o] = k;
    if (V) vout[o] = s_v[j];
  }
}

// exclusive scan of each pass's 256-bin histogram (one block of 256 threads per pass)
__global__ void __launch_bounds__(RS_THREADS) k_os_scan(const u32* __restrict__ ghist, u32* __restrict__ gbase) {
  pdl_begin();
  __shared__ u32 tot;
  u32 v = ghist[blockIdx.x * 256 + threadIdx.x];
  gbase[blockIdx.x * 256 + threadIdx.x] = block_excl_scan<u32, RS_THREADS>(v, &tot);
}

static size_t al256(size_t b) { return (b + 255) / 256 * 256; }

size_t radix_sort_temp_bytes(u64 n, bool with_vals, int nbits) {
  u64 ntiles = (n + RS_TILE - 1) / RS_TILE;
  const u64 np = (u64)(std::max(1, std::min(nbits, 8 * OS_MAX_PASSES)) + 7) / 8;
  size_t b = al256(n * 8);                       // alt keys
  if (with_vals) b += al256(n * 4);              // alt vals
  b += al256(np * ntiles * 256 * 8);             // look-back status words, one set per pass
  b += al256(OS_MAX_PASSES * 256 * 4) * 2;       // histograms, bases
  b += 256;                                      // tile counters, one per pass
  return b;
}

u64* radix_sort_keys_input(u64* keys, u64 n, int nbits, void* temp) {
  if (n <= 1 || nbits <= 0) return keys;
  const int npass = (std::min(nbits, 8 * OS_MAX_PASSES) + 7) / 8;
  (void)n;
  return (npass & 1) ? (u64*)temp : keys;  // the alternate key buffer leads the temp block
}

// scratch layout shared by radix_sort_prepare and radix_sort
struct RsLayout {
  u64* kalt; u32* valt; u64* status; u32* ghist; u32* tile_counter; u32* gbase;
};
static RsLayout rs_layout(u64 n, bool with_vals, int npass, void* temp) {
  u64 ntiles = (n + RS_TILE - 1) / RS_TILE;
  char* t = (char*)temp;
  RsLayout L;
  L.kalt = (u64*)t; t += al256(n * 8);
  L.valt = nullptr;
  if (with_vals) { L.valt = (u32*)t; t += al256(n * 4); }
  // status words (one set per pass) | histograms | tile counters (one per pass) | digit bases:
  // the first three are zeroed by ONE memset for the whole sort
  L.status = (u64*)t; t += al256((u64)npass * ntiles * 256 * 8);  // as radix_sort_temp_bytes(nbits)
  L.ghist = (u32*)t; t += al256(OS_MAX_PASSES * 256 * 4);
  L.tile_counter = (u32*)t; t += 256;
  L.gbase = (u32*)t;
  return L;
}

u32* radix_sort_prepare(u64 n, bool with_vals, int nbits, void* temp, cudaStream_t s) {
  if (nbits > 8 * OS_MAX_PASSES) nbits = 8 * OS_MAX_PASSES;
  const int npass = (std::max(nbits, 1) + 7) / 8;
  RsLayout L = rs_layout(n, with_vals, npass, temp);
  if (cudaMemsetAsync(L.status, 0, (size_t)((char*)L.gbase - (char*)L.status), s) != cudaSuccess) return nullptr;
  return L.ghist;
}

int radix_sort(u64* keys, u32* vals, u64 n, int nbits, void* temp, cudaStream_t s, int* passes,
               bool keys_in_alt, bool prepared) {
  if (passes) *passes = 0;
  if (n <= 1 || nbits <= 0) {
    if (keys_in_alt && n) launch_copy(keys, temp, n * 8, s);
    return SIEVE_OK;
  }
  if (nbits > 8 * OS_MAX_PASSES) nbits = 8 * OS_MAX_PASSES;
  const int npass = (nbits + 7) / 8;
  u64 ntiles = (n + RS_TILE - 1) / RS_TILE;
  RsLayout L = rs_layout(n, vals != nullptr, npass, temp);
  u64* kalt = L.kalt; u32* valt = L.valt; u64* status = L.status; u32* ghist = L.ghist;
  u32* tile_counter = L.tile_counter; u32* gbase = L.gbase;
  if (!prepared) {
    SV_CUDA(cudaMemsetAsync(status, 0, (size_t)((char*)gbase - (char*)status), s));
    size_t hsmem = (size_t)(RS_WARPS / 2) * npass * 256 * 4;
    SV_CUDA(sv_smem_attr(k_os_hist, (int)hsmem));
    u64 hgrid = std::min<u64>((n + RS_THREADS - 1) / RS_THREADS, (u64)sv_num_sms() * 4);
    SV_LAUNCH(k_os_hist, (unsigned)hgrid, RS_THREADS, hsmem, s)(keys_in_alt ? kalt : keys, n, npass,
                                                              nbits >= 64 ? ~0ull : (1ull << nbits) - 1, ghist);
  }
  // digit bases on the device (no host round trip): every pass runs -- a pass over a digit
  // that is constant across all keys is a stable identity permutation, so skipping it would only
  // save time, never change the result
  SV_LAUNCH(k_os_scan, npass, RS_THREADS, 0, s)(ghist, gbase);
  size_t smem = (size_t)RS_TILE * (vals ? 8 + 4 : 8);
  SV_CUDA(sv_smem_attr(k_os_pass<true>, RS_TILE * (8 + 4)));
  SV_CUDA(sv_smem_attr(k_os_pass<false>, RS_TILE * 8));
  u64* kin = keys; u32* vin = vals; u64* kout = kalt; u32* vout = valt;
  if (keys_in_alt) { kin = kalt; kout = keys; }  // keys-only: the producer wrote the alt buffer
  for (int p = 0; p < npass; p++) {
    // digits above nbits are masked off (keys may carry payload bits there)
    const u32 dmask = 8 * p + 8 <= nbits ? 255u : (1u << (nbits - 8 * p)) - 1u;
    u64* st = status + (u64)p * ntiles * 256;
    if (vals)
      SV_LAUNCH(k_os_pass<true>, (unsigned)ntiles, RS_THREADS, smem, s)(kin, vin, n, 8 * p, dmask, gbase + p * 256,
                                                                     st, tile_counter + p, kout, vout);
    else
      SV_LAUNCH(k_os_pass<false>, (unsigned)ntiles, RS_THREADS, smem, s)(kin, vin, n, 8 * p, dmask, gbase + p * 256,
                                                                      st, tile_counter + p, kout, vout);
    u64* tk = kin; kin = kout; kout = tk;
    u32* tv = vin; vin = vout; vout = tv;
    if (passes) (*passes)++;
  }
  if (kin != keys) {
    launch_copy(keys, kin, n * 8, s);
    if (vals) launch_copy(vals, vin, n * 4, s);
  }
  SV_CUDA(cudaGetLastError());
  return SIEVE_OK;
}
