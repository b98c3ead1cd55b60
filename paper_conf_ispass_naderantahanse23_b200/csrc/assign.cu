// assign.cu -- pass B: assign every invocation to its stratum and gather, per (stratum, CTA
// size), the count and the first-chronological invocation id; then pick each stratum's
// representative (footnote P:103):
//   Tier-1: the first-chronological invocation;
//   Tier-2/3: the first-chronological invocation with the most dominant CTA size
//             (max count; a tie goes to the CTA size seen first, A17).
//
// B200 design: one coalesced pass (kernel id, x, CTA in; stratum id out).  Stratum lookup is a
// per-kernel table plus a branch-free binary search over the kernel's stratum lower bounds.
// (stratum, CTA) statistics are block-private in shared memory: two fixed slots per stratum
// (k_assign_slots; a third CTA size of a stratum goes to the global table directly) or, when
// the slots do not fit, an open-addressing hash table (k_assign; 64-bit CAS only on first
// insertion) flushed when three-quarters full; native 32-bit atomics for counts and first
// offsets.  Both end in an L2-resident global table at the end of the block's range.
// The global table's contents (not its slot order) are deterministic; entries are compacted,
// gathered across ranks, radix-sorted by key and reduced, so the result is identical for any
// number of ranks or blocks.
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>

#include "kernels.cuh"

#define AS_THREADS 1024
#ifndef AS_PIPE
#define AS_PIPE 1           // the next tile's rows are loaded while this tile is processed
#endif                      // (A/B on C4: 0.96 -> 0.73 ms against 8 rows per thread unpipelined)
#ifndef AS_IPT
#define AS_IPT (AS_PIPE ? 4 : 8)
#endif
#define AS_HC 8192          // shared hash capacity (entries): 128 KB, one block per SM
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
//
// W > 0: a slot front.  Every stratum owns W fixed slots {CTA size, count, first offset} in
// shared memory; a row reads its stratum's W CTA sizes with one vector load and adds to the
// matching slot, a CTA size seen for the first time claims a free slot with a 32-bit CAS, and
// only rows whose CTA size finds no slot go to the (then small) hash table.  The slots need no
// probing (the hash alone makes a warp wait for the longest probe sequence among its lanes) and
// no flushing; a block's slots go to the L2 table once, at the end.  Every path adds the same
// (key, count, first) contributions, so the L2 table's contents are identical.
#define AS_TAB_BUDGET (96 * 1024)
#define AS_EMPTY32 0xFFFFFFFFu
#define AS_SMEM_MAX (227 * 1024 - 1024)
#ifndef AS_SLOT_IPT
#define AS_SLOT_IPT 2       // rows per thread per tile with the slot front (A/B on C4: 1 0.56, 2 0.495,
#endif                      // 3 0.50, 4 0.51, 6 0.72, 8 0.92 ms: rows in flight compete for L1 room)
template <bool SMEM_TAB, int W>
__global__ void __launch_bounds__(AS_THREADS)
k_assign(const u32* __restrict__ kid, const u64* __restrict__ x, const u32* __restrict__ cta,
         u64 n, u64 first_id, const KTab* __restrict__ g_ktab, const u64* __restrict__ g_lows,
         u32 K, u32 nlows, u32 ns, u32 hcap, u32* __restrict__ sid_out, GHash gh, u64* errflags) {
  constexpr int IPT = W > 0 ? AS_SLOT_IPT : AS_IPT;
  pdl_begin();
  extern __shared__ __align__(16) unsigned char smem[];
  const u32 nslot = W > 0 ? ns * W : 0u;
  // slots: CTA sizes stratum-major (one vector load reads a stratum's W sizes); counts and first
  // offsets slot-major, so the atomics of distinct strata fall into distinct banks
  u32* sc = (u32*)smem;                       // [ns][W] CTA sizes (AS_EMPTY32: free)
  u32* sn = sc + nslot;                       // [W][ns] counts
  u32* sf = sn + nslot;                       // [W][ns] first offsets in the block's range
  u64* hk = (u64*)(smem + ((3ull * nslot * 4 + 15) & ~15ull));   // [hcap]
  u32* hc = (u32*)(hk + hcap);                // [hcap]
  u32* hf = hc + hcap;                        // [hcap]
  KTab* s_ktab = (KTab*)(hf + hcap);          // [K]       (SMEM_TAB)
  u64* s_lows = (u64*)(s_ktab + K);           // [nlows]   (SMEM_TAB)
  const KTab* ktab = SMEM_TAB ? s_ktab : g_ktab;
  const u64* lows = SMEM_TAB ? s_lows : g_lows;
  const u32 hmask = hcap - 1, hflush = 3 * hcap / 4;   // flush to the L2 table when this full
  __shared__ u32 s_fill;
  if (SMEM_TAB) {
    for (u32 i = threadIdx.x; i < K; i += AS_THREADS) s_ktab[i] = g_ktab[i];
    for (u32 i = threadIdx.x; i < nlows; i += AS_THREADS) s_lows[i] = g_lows[i];
  }
  if constexpr (W > 0)
    for (u32 i = threadIdx.x; i < nslot; i += AS_THREADS) { sc[i] = AS_EMPTY32; sn[i] = 0; sf[i] = AS_EMPTY32; }
  for (u32 i = threadIdx.x; i < hcap; i += AS_THREADS) { hk[i] = HASH_EMPTY; hc[i] = 0; hf[i] = 0xFFFFFFFFu; }
  if (threadIdx.x == 0) s_fill = 0;
  __syncthreads();
  // n < 2^32 (sieve_load_trace): every index of the pass is a 32-bit offset
  const u32 n32 = (u32)n;
  const u32 chunk = (u32)((n + gridDim.x - 1) / gridDim.x);
  const u32 b0 = blockIdx.x * chunk;
  const u32 b1 = (u64)b0 + chunk < n32 ? b0 + chunk : n32;
  const u32 tile = AS_THREADS * IPT;
  u32 kk[IPT], cc[IPT];
  u64 vv[IPT];
  u32 tiles_done = 0, next_check = 1, last_fill = 0, last_check = 0;
  auto load_tile = [&](u32 base, u32* k_, u64* v_, u32* c_) {
#pragma unroll
    for (int j = 0; j < IPT; j++) {
      const u32 i = base + j * AS_THREADS + threadIdx.x;
      const bool ok = i < b1;
      k_[j] = ok ? __ldcs(kid + i) : 0u;
      v_[j] = ok ? __ldcs(x + i) : 0ull;
      c_[j] = (ok && cta) ? __ldcs(cta + i) : 0u;
    }
  };
#if AS_PIPE
  if (b0 < b1) load_tile(b0, kk, vv, cc);
#endif
  for (u32 base = b0; base < b1; base += tile) {
#if AS_PIPE
    u32 nk[IPT], nc[IPT];
    u64 nv[IPT];
    load_tile(base + tile, nk, nv, nc);   // in flight while this tile is processed
#else
    load_tile(base, kk, vv, cc);          // the tile's loads first, then the atomics
#endif
    KTab kts[IPT];  // per-kernel table rows, all requested before use
#pragma unroll
    for (int j = 0; j < IPT; j++) kts[j] = ktab[kk[j]];
#pragma unroll
    for (int j = 0; j < IPT; j++) {
      const u32 i = base + j * AS_THREADS + threadIdx.x;
      if (i >= b1) continue;
      const u64 v = vv[j];
      const KTab kt = kts[j];
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
      const u32 c = cc[j];
      const u32 rel = i - b0;
      if constexpr (W > 0) {
        const u32 b = sid * W;
        int slot;
        if constexpr (W == 4) {
          const uint4 k4 = *(const uint4*)(sc + b);
          slot = k4.x == c ? 0 : k4.y == c ? 1 : k4.z == c ? 2 : k4.w == c ? 3 : -1;
        } else {
          const uint2 k2 = *(const uint2*)(sc + b);
          slot = k2.x == c ? 0 : k2.y == c ? 1 : -1;
        }
        if (slot < 0 && c != AS_EMPTY32) {  // first sight of this CTA size (in the read above)
#pragma unroll
          for (int q = 0; q < W; q++) {
            const u32 cur = atomicCAS(sc + b + q, AS_EMPTY32, c);
            if (cur == AS_EMPTY32 || cur == c) { slot = q; break; }
          }
        }
        if (slot >= 0) {
          const u32 e = slot * ns + sid;
          atomicAdd(sn + e, 1u);
          if (*(volatile u32*)(sf + e) > rel) atomicMin(sf + e, rel);  // rarely lowers it
          continue;
        }
      }
      const u64 key = ((u64)sid << 32) | c;
      u32 h = hash_key(key) & hmask;
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
        h = (h + 1) & hmask;
      }
      if (!done) ghash_update(gh, key, 1, first_id + i, errflags);
    }
    const bool last = base + tile >= b1;
    ++tiles_done;
    // the fill check needs block barriers, so it runs only as often as the table's growth needs:
    // after half the tiles the last interval's growth rate would take to reach the flush level,
    // at most AS_CHECK tiles apart (a full table only sends rows to the L2 table directly, it is
    // never wrong)
    if (tiles_done < next_check && !last) {
#if AS_PIPE
#pragma unroll
      for (int j = 0; j < IPT; j++) { kk[j] = nk[j]; vv[j] = nv[j]; cc[j] = nc[j]; }
#endif
      continue;
    }
    __syncthreads();
    const u32 fill = s_fill;  // one snapshot for the whole block: nobody inserts until all read it
    __syncthreads();
    {
      const u32 grow = (fill > last_fill ? fill - last_fill : 0u) / max(1u, tiles_done - last_check);
      const u32 room = fill < hflush ? hflush - fill : 0u;
      const u32 k = grow ? room / (2u * grow) : (u32)AS_CHECK;
      next_check = tiles_done + max(1u, min(k, (u32)AS_CHECK));
      last_fill = fill;
      last_check = tiles_done;
    }
    if (fill > hflush || last) {  // rows that find no slot go to the L2 table directly
      for (u32 e = threadIdx.x; e < hcap; e += AS_THREADS) {
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
    for (int j = 0; j < IPT; j++) { kk[j] = nk[j]; vv[j] = nv[j]; cc[j] = nc[j]; }
#endif
  }
  if constexpr (W > 0) {  // the slots, once (every thread passed the last tile's barriers above)
    for (u32 e = threadIdx.x; e < nslot; e += AS_THREADS) {
      const u32 c = sc[e], sid = e / W, f = (e % W) * ns + sid;
      if (c != AS_EMPTY32 && sn[f]) ghash_update(gh, ((u64)sid << 32) | c, sn[f], first_id + b0 + sf[f], errflags);
    }
  }
}

static size_t assign_smem(u32 W, u32 ns, u32 hcap, bool smem_tab, u32 K, u32 nlows) {
  return ((3ull * ns * W * 4 + 15) & ~15ull) + (size_t)hcap * 16 +
         (smem_tab ? (size_t)K * sizeof(KTab) + (size_t)nlows * 8 : 0);
}

template <bool SMEM_TAB, int W>
static void launch_assign_v(const u32* kid, const u64* x, const u32* cta, u64 n, u64 first_id,
                            const KTab* ktab, const u64* lows, u32 K, u32 nlows, u32 ns, u32 hcap,
                            u32* sid_out, GHash gh, u64* errflags, int grid, cudaStream_t s) {
  const size_t sm = assign_smem(W, ns, hcap, SMEM_TAB, K, nlows);
  sv_smem_attr(k_assign<SMEM_TAB, W>, (int)sm);
  SV_LAUNCH((k_assign<SMEM_TAB, W>), grid, AS_THREADS, sm, s)(kid, x, cta, n, first_id, ktab, lows, K, nlows,
                                                              ns, hcap, sid_out, gh, errflags);
}

// Variant choice: the slot front with a small hash behind it (2 slots per stratum, a 2,048-entry
// hash, or 1,024 / 512 entries when that is what fits) in AS_SLOT_BUDGET of shared memory, else
// the 8,192-entry hash alone (A/B
// on C4: slots + 512 / 1,024 / 2,048 / 4,096 hash entries 0.49 ms each; four slots per stratum
// 0.67 ms -- the 16-byte key reads and the stride-4 atomics conflict; the hash alone 0.57 ms, on
// C5 9.35 ms).  Without the hash behind them, slots that overflow send rows to contended L2
// atomics (C5, five CTA sizes per stratum: 87 ms).  Test hook SIEVE_ASSIGN: "hash" forces the
// hash alone, "4" four slots per stratum.
#ifndef AS_SLOT_BUDGET
#define AS_SLOT_BUDGET (220 * 1024)
#endif
#ifndef AS_SLOT_HASH
#define AS_SLOT_HASH 2048   // the hash behind the slots: this size, or the largest of 1,024 / 512
#endif                      // that fits the budget (C5's 5,566 strata: 1,024 entries, 9.37 -> 6.95 ms)
void launch_assign(const u32* kid, const u64* x, const u32* cta, u64 n, u64 first_id,
                   const KTab* ktab, const u64* lows, u32 K, u32 nlows, u32 ns, u32* sid_out, GHash gh,
                   u64* errflags, int grid, cudaStream_t s) {
  if (n == 0) return;
  u64 maxgrid = (n + (u64)AS_THREADS * AS_SLOT_IPT - 1) / ((u64)AS_THREADS * AS_SLOT_IPT);
  if ((u64)grid > maxgrid) grid = (int)maxgrid;
  const char* force = getenv("SIEVE_ASSIGN");
  const bool hash_only = force && !strcmp(force, "hash");
  const bool w4 = force && !strcmp(force, "4");
  const size_t tab = (size_t)K * sizeof(KTab) + (size_t)nlows * 8;
  if (!hash_only && tab <= AS_TAB_BUDGET) {
    if (w4 && assign_smem(4, ns, AS_SLOT_HASH, true, K, nlows) <= AS_SMEM_MAX) {
      launch_assign_v<true, 4>(kid, x, cta, n, first_id, ktab, lows, K, nlows, ns, AS_SLOT_HASH, sid_out, gh,
                               errflags, grid, s);
      return;
    }
    if (!w4)
      for (u32 hc = AS_SLOT_HASH; hc >= 512; hc >>= 1)
        if (assign_smem(2, ns, hc, true, K, nlows) <= AS_SLOT_BUDGET) {
          launch_assign_v<true, 2>(kid, x, cta, n, first_id, ktab, lows, K, nlows, ns, hc, sid_out, gh,
                                   errflags, grid, s);
          return;
        }
  }
  if (tab <= AS_TAB_BUDGET)
    launch_assign_v<true, 0>(kid, x, cta, n, first_id, ktab, lows, K, nlows, ns, AS_HC, sid_out, gh, errflags,
                             grid, s);
  else
    launch_assign_v<false, 0>(kid, x, cta, n, first_id, ktab, lows, K, nlows, ns, AS_HC, sid_out, gh, errflags,
                              grid, s);
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
