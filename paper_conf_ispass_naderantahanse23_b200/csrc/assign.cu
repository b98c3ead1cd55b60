// assign.cu -- pass B: assign every invocation to its stratum and gather, per (stratum, CTA
// size), the count and the first-chronological invocation id; then pick each stratum's
// representative (footnote P:103):
//   Tier-1: the first-chronological invocation;
//   Tier-2/3: the first-chronological invocation with the most dominant CTA size
//             (max count; a tie goes to the CTA size seen first, A17).
//
// B200 design: one coalesced pass (kernel id, x, CTA in; stratum id out).  Stratum lookup is a
// per-kernel table plus a branch-free binary search over the kernel's stratum lower bounds.
// (stratum, CTA) statistics use a block-private open-addressing hash table in shared memory
// (native 32-bit atomics for counts and first offsets; 64-bit CAS only on first insertion),
// flushed into an L2-resident global table when half full and at the end of the block's range.
// The global table's contents (not its slot order) are deterministic; entries are compacted,
// gathered across ranks, radix-sorted by key and reduced, so the result is identical for any
// number of ranks or blocks.
#include <algorithm>
#include <cstdint>

#include "kernels.cuh"

#define AS_THREADS 1024
#ifndef AS_PIPE
#define AS_PIPE 1           // the next tile's rows are loaded while this tile is processed
#endif                      // (A/B on C4: 0.96 -> 0.73 ms against 8 rows per thread unpipelined)
#ifndef AS_IPT
#define AS_IPT (AS_PIPE ? 4 : 8)
#endif
#define AS_HC 8192          // shared hash capacity (entries): 128 KB, one block per SM
#define AS_FLUSH (3 * AS_HC / 4)      // flush to the L2 table when this full
#define AS_MAXP 32          // probes before falling back to the global table
#ifndef AS_CHECK
#define AS_CHECK 32         // at most this many tiles between the fill checks (A/B, C4 / C5:
                            // every tile 0.73 / 10.7 ms, growth-paced up to 8: 0.59, 32: 0.57 / 10.0)
#endif

// One block per SM with a large table: a block's contiguous chunk sees nearly every (stratum,
// CTA) pair of the trace (thousands), so a small table would flush -- i.e. issue contended L2
// atomics on the same hot keys from every block -- many times per block.
int assign_grid() { return sv_num_sms(); }

__device__ __forceinline__ u32 hash_key(u64 k) {
  return (u32)((k * 0x9E3779B97F4A7C15ull) >> 32);
}

__device__ void ghash_update(GHash gh, u64 key, u64 cnt, u64 first, u64* errflags) {
  u64 h = (u64)hash_key(key) & (gh.cap - 1);
  for (u64 probe = 0; probe < gh.cap; probe++) {
    u64 cur = gh.keys[h];
    if (cur == HASH_EMPTY) {
      cur = atomicCAS((unsigned long long*)&gh.keys[h], HASH_EMPTY, key);
      if (cur == HASH_EMPTY) cur = key;
    }
    if (cur == key) {
      atomicAdd((unsigned long long*)&gh.cnt[h], (unsigned long long)cnt);
      atomicMin((unsigned long long*)&gh.first[h], (unsigned long long)first);
      return;
    }
    h = (h + 1) & (gh.cap - 1);
  }
  atomicMax((unsigned long long*)&errflags[2], 1ull);  // global table full: caller retries bigger
}

// SMEM_TAB: the per-kernel table and the strata lower bounds are staged in shared memory next
// to the hash (every row looks them up; from global memory the dependent loads of the binary
// search and the LSU queue were the kernel's main stalls)
#define AS_TAB_BUDGET (96 * 1024)
template <bool SMEM_TAB>
__global__ void __launch_bounds__(AS_THREADS)
k_assign(const u32* __restrict__ kid, const u64* __restrict__ x, const u32* __restrict__ cta,
         u64 n, u64 first_id, const KTab* __restrict__ g_ktab, const u64* __restrict__ g_lows,
         u32 K, u32 nlows, u32* __restrict__ sid_out, GHash gh, u64* errflags) {
  pdl_begin();
  extern __shared__ __align__(16) unsigned char smem[];
  u64* hk = (u64*)smem;              // [AS_HC]
  u32* hc = (u32*)(hk + AS_HC);      // [AS_HC]
  u32* hf = hc + AS_HC;              // [AS_HC]
  KTab* s_ktab = (KTab*)(hf + AS_HC);          // [K]       (SMEM_TAB)
  u64* s_lows = (u64*)(s_ktab + K);             // [nlows]   (SMEM_TAB)
  const KTab* ktab = SMEM_TAB ? s_ktab : g_ktab;
  const u64* lows = SMEM_TAB ? s_lows : g_lows;
  __shared__ u32 s_fill;
  if (SMEM_TAB) {
    for (u32 i = threadIdx.x; i < K; i += AS_THREADS) s_ktab[i] = g_ktab[i];
    for (u32 i = threadIdx.x; i < nlows; i += AS_THREADS) s_lows[i] = g_lows[i];
  }
  for (u32 i = threadIdx.x; i < AS_HC; i += AS_THREADS) { hk[i] = HASH_EMPTY; hc[i] = 0; hf[i] = 0xFFFFFFFFu; }
  if (threadIdx.x == 0) s_fill = 0;
  __syncthreads();
  u64 chunk = (n + gridDim.x - 1) / gridDim.x;
  u64 b0 = (u64)blockIdx.x * chunk;
  u64 b1 = b0 + chunk < n ? b0 + chunk : n;
  const u64 tile = (u64)AS_THREADS * AS_IPT;
  u32 kk[AS_IPT], cc[AS_IPT];
  u64 vv[AS_IPT];
  u32 tiles_done = 0, next_check = 1, last_fill = 0, last_check = 0;
  auto load_tile = [&](u64 base, u32* k_, u64* v_, u32* c_) {
#pragma unroll
    for (int j = 0; j < AS_IPT; j++) {
      u64 i = base + (u64)j * AS_THREADS + threadIdx.x;
      bool ok = i < b1;
      k_[j] = ok ? __ldcs(kid + i) : 0u;
      v_[j] = ok ? __ldcs(x + i) : 0ull;
      c_[j] = (ok && cta) ? __ldcs(cta + i) : 0u;
    }
  };
#if AS_PIPE
  load_tile(b0, kk, vv, cc);
#endif
  for (u64 base = b0; base < b1; base += tile) {
#if AS_PIPE
    u32 nk[AS_IPT], nc[AS_IPT];
    u64 nv[AS_IPT];
    load_tile(base + tile, nk, nv, nc);   // in flight while this tile is processed
#else
    load_tile(base, kk, vv, cc);          // the tile's loads first, then the atomics
#endif
    KTab kts[AS_IPT];  // per-kernel table rows (L1-resident), all requested before use
#pragma unroll
    for (int j = 0; j < AS_IPT; j++) kts[j] = ktab[kk[j]];
#pragma unroll
    for (int j = 0; j < AS_IPT; j++) {
      u64 i = base + (u64)j * AS_THREADS + threadIdx.x;
      if (i >= b1) continue;
      u64 v = vv[j];
      KTab kt = kts[j];
      u32 sid = kt.base;
      if (kt.m > 1) {  // number of lower bounds lows[1..m) that are <= v
        const u64* L = lows + kt.lows_off;
        u32 lo = 0, cnt = kt.m - 1;
        while (cnt > 0) {
          u32 half = cnt >> 1;
          if (L[lo + half] <= v) { lo += half + 1; cnt -= half + 1; } else cnt = half;
        }
        sid += lo;
      }
      if (sid_out) sid_out[i] = sid;
      u32 c = cc[j];
      u64 key = ((u64)sid << 32) | c;
      u32 rel = (u32)(i - b0);
      u32 h = hash_key(key) & (AS_HC - 1);
      bool done = false;
      for (int p = 0; p < AS_MAXP; p++) {
        u64 cur = hk[h];
        if (cur == HASH_EMPTY) {
          cur = atomicCAS((unsigned long long*)&hk[h], HASH_EMPTY, key);
          if (cur == HASH_EMPTY) { atomicAdd(&s_fill, 1u); cur = key; }
        }
        if (cur == key) {
          atomicAdd(&hc[h], 1u);
          if (*(volatile u32*)&hf[h] > rel) atomicMin(&hf[h], rel);  // rarely lowers it
          done = true;
          break;
        }
        h = (h + 1) & (AS_HC - 1);
      }
      if (!done) ghash_update(gh, key, 1, first_id + i, errflags);
    }
    bool last = base + tile >= b1;
    ++tiles_done;
    // the fill check needs block barriers, so it runs only as often as the table's growth needs:
    // after half the tiles the last interval's growth rate would take to reach the flush level,
    // at most AS_CHECK tiles apart (a full table only sends rows to the L2 table directly, it is
    // never wrong)
    if (tiles_done < next_check && !last) {
#if AS_PIPE
#pragma unroll
      for (int j = 0; j < AS_IPT; j++) { kk[j] = nk[j]; vv[j] = nv[j]; cc[j] = nc[j]; }
#endif
      continue;
    }
    __syncthreads();
    const u32 fill = s_fill;  // one snapshot for the whole block: nobody inserts until all read it
    __syncthreads();
    {
      const u32 grow = (fill > last_fill ? fill - last_fill : 0u) / max(1u, tiles_done - last_check);
      const u32 room = fill < AS_FLUSH ? AS_FLUSH - fill : 0u;
      const u32 k = grow ? room / (2u * grow) : (u32)AS_CHECK;
      next_check = tiles_done + max(1u, min(k, (u32)AS_CHECK));
      last_fill = fill;
      last_check = tiles_done;
    }
    if (fill > AS_FLUSH || last) {  // rows that find no slot go to the L2 table directly
      for (u32 e = threadIdx.x; e < AS_HC; e += AS_THREADS) {
        u64 key = hk[e];
        if (key != HASH_EMPTY) {
          ghash_update(gh, key, hc[e], first_id + b0 + hf[e], errflags);
          hk[e] = HASH_EMPTY; hc[e] = 0; hf[e] = 0xFFFFFFFFu;
        }
      }
      __syncthreads();
      if (threadIdx.x == 0) s_fill = 0;
      last_fill = 0;
      __syncthreads();
    }
#if AS_PIPE
#pragma unroll
    for (int j = 0; j < AS_IPT; j++) { kk[j] = nk[j]; vv[j] = nv[j]; cc[j] = nc[j]; }
#endif
  }
}

void launch_assign(const u32* kid, const u64* x, const u32* cta, u64 n, u64 first_id,
                   const KTab* ktab, const u64* lows, u32 K, u32 nlows, u32* sid_out, GHash gh,
                   u64* errflags, int grid, cudaStream_t s) {
  if (n == 0) return;
  size_t smem = (size_t)AS_HC * (8 + 4 + 4);
  size_t tab = (size_t)K * sizeof(KTab) + (size_t)nlows * 8;
  u64 maxgrid = (n + (u64)AS_THREADS * AS_IPT - 1) / ((u64)AS_THREADS * AS_IPT);
  if ((u64)grid > maxgrid) grid = (int)maxgrid;
  if (tab <= AS_TAB_BUDGET) {
    sv_smem_attr(k_assign<true>, (int)(smem + tab));
    SV_LAUNCH(k_assign<true>, grid, AS_THREADS, smem + tab, s)(kid, x, cta, n, first_id, ktab, lows, K,
                                                                nlows, sid_out, gh, errflags);
  } else {
    sv_smem_attr(k_assign<false>, (int)smem);
    SV_LAUNCH(k_assign<false>, grid, AS_THREADS, smem, s)(kid, x, cta, n, first_id, ktab, lows, K,
                                                           nlows, sid_out, gh, errflags);
  }
}

__global__ void k_hash_compact(GHash gh, u64* okey, u64* ocnt, u64* ofirst,
                               unsigned long long* count) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  bool occ = i < gh.cap && gh.keys[i] != HASH_EMPTY;
  u32 m = __ballot_sync(0xffffffffu, occ);
  unsigned long long base = 0;
  if (lane_id() == 0 && m) base = atomicAdd(count, (unsigned long long)__popc(m));
  base = __shfl_sync(0xffffffffu, base, 0);
  if (occ) {
    u64 o = base + __popc(m & ((1u << lane_id()) - 1u));
    okey[o] = gh.keys[i];
    ocnt[o] = gh.cnt[i];
    ofirst[o] = gh.first[i];
  }
}

void launch_hash_compact(GHash gh, u64* okey, u64* ocnt, u64* ofirst, unsigned long long* count,
                         cudaStream_t s) {
  SV_LAUNCH(k_hash_compact, div_up(gh.cap, 256), 256, 0, s)(gh, okey, ocnt, ofirst, count);
}

__global__ void k_iota_u32(u32* p, u64 n) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = (u32)i;
}
void launch_iota_u32(u32* p, u64 n, cudaStream_t s) {
  if (n) SV_LAUNCH(k_iota_u32, div_up(n, 256), 256, 0, s)(p, n);
}

// stratum id of every compacted (stratum, CTA) entry; neutral slots (key ~0) map to ns
__global__ void k_entry_sids(const u64* key, u64 n, u32 ns, u64* out) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) { u64 s = key[i] >> 32; out[i] = s < ns ? s : ns; }
}
void launch_entry_sids(const u64* key, u64 n, u32 ns, u64* out, cudaStream_t s) {
  if (n) SV_LAUNCH(k_entry_sids, div_up(n, 256), 256, 0, s)(key, n, ns, out);
}

__global__ void k_gather_u64(const u64* src, const u32* idx, u64 n, u64* dst) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) dst[i] = src[idx[i]];
}
void launch_gather_u64(const u64* src, const u32* idx, u64 n, u64* dst, cudaStream_t s) {
  if (n) SV_LAUNCH(k_gather_u64, div_up(n, 256), 256, 0, s)(src, idx, n, dst);
}

// one thread per stratum over its (sorted) entries; equal keys (from different ranks) merge
__global__ void k_reps(const u64* key, const u64* cnt, const u64* first, u64 E, const u32* tier,
                       u32 nstrata, u64* rep_id, u64* rep_cta) {
  pdl_begin();
  u32 s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= nstrata) return;
  u64 lo = 0, hi = E;
  u64 kv = (u64)s << 32;
  while (lo < hi) { u64 m = (lo + hi) >> 1; if (key[m] < kv) lo = m + 1; else hi = m; }
  u64 best_c = 0, best_f = ~0ull, best_k = 0;   // dominant CTA (count desc, first asc)
  u64 min_f = ~0ull, min_k = 0;                 // first-chronological overall
  u64 i = lo;
  while (i < E && (key[i] >> 32) == s) {
    u64 k = key[i], c = 0, f = ~0ull;
    while (i < E && key[i] == k) { c += cnt[i]; f = first[i] < f ? first[i] : f; i++; }
    if (c > best_c || (c == best_c && f < best_f)) { best_c = c; best_f = f; best_k = k; }
    if (f < min_f) { min_f = f; min_k = k; }
  }
  if (tier[s] == 1) { rep_id[s] = min_f; rep_cta[s] = min_k & 0xFFFFFFFFull; }
  else { rep_id[s] = best_f; rep_cta[s] = best_k & 0xFFFFFFFFull; }
}

void launch_reps(const u64* key, const u64* cnt, const u64* first, u64 E, const u32* tier,
                 u32 nstrata, u64* rep_id, u64* rep_cta, cudaStream_t s) {
  if (nstrata) SV_LAUNCH(k_reps, div_up(nstrata, 128), 128, 0, s)(key, cnt, first, E, tier, nstrata, rep_id, rep_cta);
}

__global__ void k_rep_xy(const u64* rep_id, u32 nstrata, u64 first_id, u64 n_local, const u64* x,
                         const u64* y, u64* out) {
  pdl_begin();
  u32 s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= nstrata) return;
  u64 r = rep_id[s];
  bool mine = r >= first_id && r - first_id < n_local;
  out[s] = mine ? x[r - first_id] : 0;                          // [x of every stratum |
  out[nstrata + (u64)s] = (mine && y) ? y[r - first_id] : 0;    //  y of every stratum]
}

void launch_rep_xy(const u64* rep_id, u32 nstrata, u64 first_id, u64 n_local, const u64* x,
                   const u64* y, u64* out, cudaStream_t s) {
  if (nstrata) SV_LAUNCH(k_rep_xy, div_up(nstrata, 128), 128, 0, s)(rep_id, nstrata, first_id, n_local, x, y, out);
}

// ------------------------------------------------------------------------------------------
// Copies issued by the SMs instead of the copy engines: the path's small host<->device tables
// (through the pinned staging arena, which UVA maps into the device's address space) and its
// device-to-device moves.  A concurrent bulk H2D on another stream (sieve_load_trace of the next
// trace) occupies the copy engines for tens of milliseconds; copy-engine work queued behind it
// would stall every synchronisation of this call.
__global__ void k_copy_words(u32* __restrict__ dst, const u32* __restrict__ src, u64 n) {
  pdl_begin();
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) dst[i] = src[i];
}
__global__ void k_copy_bytes(unsigned char* __restrict__ dst, const unsigned char* __restrict__ src, u64 n) {
  pdl_begin();
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) dst[i] = src[i];
}
void launch_copy(void* dst, const void* src, u64 bytes, cudaStream_t s) {
  if (!bytes) return;
  if ((((uintptr_t)dst | (uintptr_t)src | bytes) & 3) == 0) {
    u64 n = bytes / 4;
    SV_LAUNCH(k_copy_words, (unsigned)std::min<u64>(div_up(n, 256), 2048), 256, 0, s)((u32*)dst, (const u32*)src, n);
  } else {
    SV_LAUNCH(k_copy_bytes, (unsigned)std::min<u64>(div_up(bytes, 256), 2048), 256, 0, s)(
        (unsigned char*)dst, (const unsigned char*)src, bytes);
  }
}

// several copies in ONE launch (blockIdx.y = region): the orchestrator's small host <-> device
// tables of one step go together (each separate copy was a launch plus a PCIe round trip)
__global__ void k_copy_multi(CopyRegions r) {
  pdl_begin();
  const int q = blockIdx.y;
  if (q >= r.k) return;
  unsigned char* d = (unsigned char*)r.dst[q];
  const unsigned char* sp = (const unsigned char*)r.src[q];
  const u64 n = r.bytes[q];
  const u64 stride = (u64)gridDim.x * blockDim.x;
  const u64 t = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if ((((uintptr_t)d | (uintptr_t)sp) & 7) == 0) {
    const u64 nw = n / 8;
    for (u64 i = t; i < nw; i += stride) ((u64*)d)[i] = ((const u64*)sp)[i];
    for (u64 i = nw * 8 + t; i < n; i += stride) d[i] = sp[i];
  } else {
    for (u64 i = t; i < n; i += stride) d[i] = sp[i];
  }
}
void launch_copy_multi(const CopyRegions& r, cudaStream_t s) {
  if (r.k <= 0) return;
  u64 mx = 0;
  for (int q = 0; q < r.k; q++) mx = r.bytes[q] > mx ? r.bytes[q] : mx;
  if (!mx) return;
  dim3 grid(std::min<u64>(div_up(mx, 256 * 8), 512), r.k);
  SV_LAUNCH(k_copy_multi, grid, 256, 0, s)(r);
}

__global__ void k_fill_u64(u64* p, u64 n, u64 v) {
  pdl_begin();
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) p[i] = v;
}
void launch_fill_u64(u64* p, u64 n, u64 v, cudaStream_t s) {
  if (n) SV_LAUNCH(k_fill_u64, min(div_up(n, 256), 4096u), 256, 0, s)(p, n, v);
}
// several fills in one launch (FILL_MAX regions): per-round buffer initialisation
__global__ void k_fill_multi(FillRegions r) {
  pdl_begin();
  for (int q = 0; q < r.k; q++)
    for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < r.n[q]; i += (u64)gridDim.x * blockDim.x)
      r.p[q][i] = r.v[q];
}
void launch_fill_multi(const FillRegions& r, cudaStream_t s) {
  u64 mx = 0;
  for (int q = 0; q < r.k; q++) mx = r.n[q] > mx ? r.n[q] : mx;
  if (mx) SV_LAUNCH(k_fill_multi, min(div_up(mx, 256), 4096u), 256, 0, s)(r);
}

__global__ void k_u128_to_limbs(const u64* src, u64 n, u64* limbs) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) limbs_from_u128(src[2 * i], src[2 * i + 1], limbs + 4 * i);
}
__global__ void k_limbs_to_u128(const u64* limbs, u64 n, u64* dst) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) limbs_to_u128(limbs + 4 * i, dst + 2 * i, dst + 2 * i + 1);
}
void launch_u128_to_limbs(const u64* src, u64 n, u64* limbs, cudaStream_t s) {
  if (n) SV_LAUNCH(k_u128_to_limbs, div_up(n, 256), 256, 0, s)(src, n, limbs);
}
void launch_limbs_to_u128(const u64* limbs, u64 n, u64* dst, cudaStream_t s) {
  if (n) SV_LAUNCH(k_limbs_to_u128, div_up(n, 256), 256, 0, s)(limbs, n, dst);
}

// MIN folded into MAX for the grouped cross-rank reductions: min(a, b) = ~max(~a, ~b)
__global__ void k_complement(u64* p, u64 n, u64 stride) {
  pdl_begin();
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x)
    p[i * stride] = ~p[i * stride];
}
void launch_complement(u64* p, u64 n, u64 stride, cudaStream_t s) {
  if (n) SV_LAUNCH(k_complement, min(div_up(n, 256), 4096u), 256, 0, s)(p, n, stride);
}

// pass B's exchange word set (one SUM all-reduce of world + 1 lanes, no host round trip before
// it): x[0] = this rank's table-overflow flag, x[1 + r] = rank r's entry count (0 elsewhere)
__global__ void k_exchange_prep(const u64* flag, const unsigned long long* count, int rank, int world, u64* x) {
  pdl_begin();
  int i = threadIdx.x;
  if (i == 0) x[0] = flag[0] ? 1ull : 0ull;
  if (i < world) x[1 + i] = i == rank ? (u64)count[0] : 0ull;
}
void launch_exchange_prep(const u64* flag, const unsigned long long* count, int rank, int world, u64* x,
                          cudaStream_t s) {
  SV_LAUNCH(k_exchange_prep, 1, ((world + 31) / 32) * 32, 0, s)(flag, count, rank, world, x);
}

// 16-bit trace columns (SIEVE_KID16 / SIEVE_CTA16) widened to the library's u32 columns
__global__ void k_widen_u16(const unsigned short* __restrict__ src, u64 n, u32* __restrict__ dst) {
  pdl_begin();
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) dst[i] = src[i];
}
void launch_widen_u16(const void* src, u64 n, u32* dst, cudaStream_t s) {
  if (n) SV_LAUNCH(k_widen_u16, (u32)std::min<u64>(div_up(n, 256), (u64)sv_num_sms() * 16), 256, 0, s)(
      (const unsigned short*)src, n, dst);
}
