// kernels.cuh -- launchers of every sm_100a kernel on the stratification path, and the small
// device-side tables they share.  See DESIGN.md section 5 for each kernel's roofline.
#pragma once
#include "common.cuh"

// ---------------- pass A: per-kernel exact moments ----------------------------------
// Per-block partial record per kernel (48 B): n, S1 (96-bit: lo + 32-bit hi), S2 (u128),
// min and max instruction count.
struct KMomPartial {
  u32 n;
  u32 s1hi;
  u64 s1lo;
  u64 s2lo, s2hi;
  u64 mn, mx;
};
// Per-kernel result of pass A (before / after the cross-rank reduction):
//   lanes[k*9 + 0] = n,  lanes[k*9 + 1..4] = S1 limbs,  lanes[k*9 + 5..8] = S2 limbs   (SUM)
//   mm[k*2 + 0] = min x (MIN), mm[k*2 + 1] = max x (MAX)
// totals: tot_lanes[0..3] = C_meas limbs (SUM); tot_max[0] = max x, tot_max[1] = error flags
#define MOM_LANES 9
#define ERRF_KID 1ull
#define ERRF_RANGE 2ull

struct MomentsScratch {
  KMomPartial* part;   // [grid][kt]
  u64* blk_tot;        // [grid][3]: C_meas lo, hi, max x
  int grid;
  u32 kt;
};
int moments_kt(u32 K);  // kernels per smem pass
int moments_grid(u32 kt);
void launch_moments(const u32* kid, const u64* x, const u64* y, u64 n, u32 K, u32 k0, u32 kt,
                    KMomPartial* part, u64* blk_tot, u64* errflags, int grid, cudaStream_t s);
void launch_moments_reduce(const KMomPartial* part, const u64* blk_tot, int grid, u32 k0, u32 kt,
                           u32 K, u64* lanes, u64* mm, u64* local_n, u64* tot_lanes, u64* tot_max,
                           bool do_totals, cudaStream_t s);

// ---------------- Tier-3 key compaction ------------------------------------------------------
// key = (t3rank(kid) << bx) + x ; t3rank = 0xFFFFFFFF for kernels not in Tier-3
void launch_t3_compact(const u32* kid, const u64* x, u64 n, const u32* t3rank, u32 bx,
                       u64* keys_out, unsigned long long* counter, cudaStream_t s);

// ---------------- LSD radix sort (u64 keys, optional u32 payload) ----------------------------
size_t radix_sort_temp_bytes(u64 n, bool with_vals, int nbits = 64);  // nbits as passed to radix_sort
// sorts keys[0..n) by bits [0, nbits) (higher bits ride along); result in keys/vals (in place via
// internal ping-pong);
// stream-ordered, no host synchronisation
int radix_sort(u64* keys, u32* vals, u64 n, int nbits, void* temp, cudaStream_t s,
               int* passes = nullptr, bool keys_in_alt = false, bool prepared = false);
// keys-only sorts: where the producer should write the n keys so that radix_sort(..., keys_in_alt
// = (returned != keys)) ends in `keys` without a copy-back (odd pass counts start in the alternate
// buffer, which leads `temp`)
u64* radix_sort_keys_input(u64* keys, u64 n, int nbits, void* temp);
// optional: zero the sort's scratch now and return its digit-histogram array (npass x 256 u32),
// for a producer that accumulates the histograms of the keys it writes; then call radix_sort
// with prepared = true (it skips its zeroing and its histogram pass)
u32* radix_sort_prepare(u64 n, bool with_vals, int nbits, void* temp, cudaStream_t s);

void scan_u32(const u32* in, u32* out, u64 n, void* temp, u32* total, cudaStream_t s);
// the calling thread's single-pass scan state (a context's persistent, zero-initialised buffer of
// SCAN_SP_MAX_TILES + 2 words; nullptr: three-kernel scans).  Set by the API entry points.
#define SCAN_SP_MAX_TILES 4096
void scan_set_state(u64* state);
size_t scan_u32_temp_bytes(u64 n);

// ---------------- KDE over open segments ([8], [36]; A6-A10) -----------------------------
struct SegDev {
  u64 lo, hi;   // value range [lo, hi] (global, replicated)
  double h, inv_h;
  double cq;    // (G - 1) / (hi - lo): cell estimate (made exact against the grid table)
  double cm;    // margin in cell units: an estimate e = rn(rn(x - lo) * cq) with
                // j + cm < e < j + 1 - cm (j < G - 1) proves g_j <= x < g_{j+1} (cell_fast)
};
// host: cm for segment [lo, hi] on a G-point grid (>= 1 disables the fast path).  With
// E = (x - lo)(G - 1)/(hi - lo) exact, |e - E| <= G 2^-52 (two roundings) and every grid point
// in cell units is within (hi + 1)(G - 1) 2^-51 / (hi - lo) of its index (A9: the product
// (hi - lo) j rounded, one division, one addition), so e in (j + cm, j + 1 - cm) puts E strictly
// between g_j and g_{j+1} (the grid is non-decreasing); cm doubles that bound.
inline double cell_margin(u64 lo, u64 hi, u32 G) {
  if (hi <= lo) return 2.0;
  const double m = 2.0 * ((double)G * 0x1p-52 + ((double)hi + 1.0) * (double)(G - 1) * 0x1p-51 / (double)(hi - lo));
  return m < 0.25 ? m : 2.0;
}
#define KDE_WC 7.54983443527075   // sqrt(57): |z| <= this <=> t <= 28.5 (in-window term count)
#ifndef KDE_TJ
#define KDE_TJ 32       // grid points per tile (32: one point per lane; 16: two value slices)
#endif
#ifndef KDE_CH
#ifndef KDE_CH
#define KDE_CH 512      // values per work item (A/B: 512 beats 256 by 2.5%; 16-point tiles lose)
#endif
#endif
// per (segment, tile of KDE_TJ grid points): the bucketed values whose cells meet the tile's
// window, split into regions by the lanes that need them (regions: kde_region_bytes(tiles)) and
// chunked into work items whose descriptors go to item_desc; tile_items[nseg * tiles] receives
// the item total
void kde_plan(const SegDev* segs, u32 nseg, u32 G, const double* gtab, const u32* off,
              void* regions, u32* tile_items, void* scan_temp, void* item_desc /* kde_item_bytes */,
              cudaStream_t s);
size_t kde_region_bytes(u64 ntiles);
// a tile has at most ceil(tile values / KDE_CH) + kde_items_per_tile_slack() work items
u32 kde_items_per_tile_slack();
size_t kde_item_bytes(u32 items);
// D[2j] accumulates the low 32-bit limbs of the item sums, D[2j + 1] the rest (both are plain
// u64 sums: several ranks may all-reduce them as they are); fix = true normalises them into the
// u128 D_j right away (else call launch_kde_fix after the cross-rank sum)
void launch_kde(const SegDev* segs, u32 nseg, u32 G, const u64* vals, u32 vshift, const void* regions,
                const u32* tile_items, void* item_desc /* kde_item_bytes(items) */, u32 items,
                u64* D /* [nseg][G][2] */, unsigned long long* evaluated, bool guard, bool fix,
                cudaStream_t s);
void launch_kde_fix(u64* D, u64 npoints, cudaStream_t s);

// ---------------- segmented sort by (open segment, grid cell) (a2) ----------------------------
// rounds > 1 read each re-opened part's range of the previous round's sorted keys in chunks of
// BK_CHUNK values: chunk c supplies outputs [c * BK_CHUNK, c * BK_CHUNK + len)
struct BucketChunk { u32 seg; u32 len; u64 begin; };
#define BK_CHUNK 2048
// max j with g[j] <= x, for lo <= x (so the answer exists); cq = (G - 1) / (hi - lo) gives the
// estimate, which is exact unless x lies within rounding error of a grid point: the two table
// entries that confirm it are loaded together (one L2 round trip), and a miss walks the table
// (g is non-decreasing in j)
__device__ __forceinline__ u32 cell_of(const double* g, u32 G, u64 lo, double cq, u64 x) {
  double xd = __ull2double_rn(x);  // exact: x < 2^44
  double e = __dmul_rn(__ull2double_rn(x - lo), cq);
  u32 j = e >= (double)(G - 1) ? G - 1 : (u32)e;
  u32 j1 = j + 1 < G ? j + 1 : j;
  double g0 = __ldg(g + j), g1 = __ldg(g + j1);
  if (g0 <= xd && (j1 == j || g1 > xd)) return j;
  while (j + 1 < G && __ldg(g + j + 1) <= xd) j++;
  while (j > 0 && __ldg(g + j) > xd) j--;
  return j;
}

// gtab[s * G + j] = g_j of segment s (A9)
void launch_grid_tab(const SegDev* segs, u32 nseg, u32 G, double* gtab, cudaStream_t s);
// out[i] = (x << ib) | idx, idx = s * G + cell(x) (ncell if x is outside [lo, hi] of segment s);
// chunks == nullptr: in = tagged Tier-3 keys (s = (key >> bx) - seg0, keys of other segments get
// the sentinel), else x = in[..] >> in_shift; *inwin += in-window KDE terms
void launch_cellkey(const BucketChunk* chunks, const u64* in, u64 nin, u32 bx, u32 in_shift,
                    const SegDev* segs, u32 G, const double* gtab, u32 ib, u32 ncell, u32 seg0,
                    u64* out, unsigned long long* inwin, u32* ghist /* nullable: radix_sort_prepare */,
                    cudaStream_t s);
// off[c] = first position of the idx-sorted keys with idx >= c, c = 0..ncell
void launch_cell_offsets(const u64* keys, u64 n, u32 ib, u32 ncell, u32* off, cudaStream_t s);

// ---- cell grouping by counting sort (bucket.cu; the default for G <= GROUP_MAXG) ----
#define GROUP_MAXG 8192
#define GROUP_CH 8192   // values per chunk (= GR_CH in bucket.cu)
#define GROUP_T3_SMEM_MAX 16384   // Tier-3 kernels the round-1 grouping counts in shared memory
// round 1: the Tier-3 rows' x grouped by t3rank at out[seg_base[t3rank] ...] (cursor zeroed)
size_t group_t3_temp_bytes(u32 n_t3);
// part (nullable): pass A's per-block partials of this trace (part_grid blocks x part_kt kernels,
// every kernel in one pass), whose per-block counts then give the output bases directly;
// t3kern[t] = the kernel of segment t (read only with part)
// n_t3: Tier-3 kernels (an upper bound when n_t3_dev != nullptr holds the live count on the
// device: the kernels may then be queued before the host knows the tiers)
void launch_group_t3(const u32* kid, const u64* x, u64 n, u32 K, const u32* t3rank, u32 n_t3,
                     const u32* n_t3_dev, const u32* seg_base, u32* cursor, u64* out,
                     void* temp /* group_t3_temp_bytes(n_t3) */, const KMomPartial* part, int part_grid,
                     u32 part_kt, const u32* t3kern, cudaStream_t s);
// tiers on the device (the same exact test as the host's): t3rank[k] (0xFFFFFFFF unless Tier-3),
// seg_base[t] = exclusive prefix of the local counts of the Tier-3 kernels in kernel order,
// t3kern[t] = kernel of segment t, counts[0] = Tier-3 kernels, counts[1] = their local rows
void launch_tiers(const u64* lanes, const u64* mm, const u64* local_n, u32 K, u32 p, u32 q, u32* t3rank,
                  u32* seg_base, u32* t3kern, u32* counts, cudaStream_t s);
// chunks (<= GROUP_CH values of one segment's source range each, the chunks of segment s are
// seg_chunk[s] .. seg_chunk[s + 1] - 1) -> out grouped by (segment, cell) with
// off[s * G + c] = first position of cell c of segment s, off[nseg * G] = values grouped
// (values outside their segment's [lo, hi] are dropped); cells [nchunks * GROUP_CH], hist / rel
// [nchunks * G], tot [nseg * G] scratch; *inwin += in-window KDE terms (nullable)
// segments of many chunks walk in groups of <= WALK_GROUP chunks (nullable: one thread per
// (segment, cell) walks all its chunks): grp[g] = {first, end chunk}, seg_grp[nseg + 1] the
// segments' group ranges, gs [ngrp * G] scratch
#define WALK_GROUP 64
#define WALK_MIN_CHUNKS 256   // the groups only when some segment has more chunks than this
struct WalkGroups { const uint2* grp; const u32* seg_grp; u32 ngrp; u32* gs; };
void launch_cell_group(const BucketChunk* chunks, u32 nchunks, const u64* src, const SegDev* segs, u32 nseg,
                       u32 G, const u32* seg_chunk, unsigned short* cells, u32* hist, u32* rel, u32* tot,
                       u32* off, void* scan_temp, u64* out, unsigned long long* inwin, cudaStream_t s,
                       const WalkGroups* wg = nullptr);

// ---------------- valleys and thresholds (A11-A13) ---------------------------------------------
// T[s*tstride + q], nt[s], kind[s] (1 = valley, 2 = bisect)
// D as the KDE leaves it (two u64 lanes per grid point: low-limb sum, rest); normalised to u128
// in place when keep_D (debug read-back) or when G is too large to stage in shared memory
void launch_valleys(const SegDev* segs, u32 nseg, u32 G, u32 shift, u64* D, u64* T,
                    u32 tstride, u32* nt, u32* kind, bool keep_D, cudaStream_t s);

// ---------------- part moments (A13 f) ----------------------------------------------------------
// parts of segment s: q = 0..nt[s]; part_off[s] = first part index (exclusive scan of nt + 1, on
// the device), part_off[nseg] = number of parts (<= cap = nseg * tstride)
void launch_part_offsets(const u32* nt, u32 nseg, u32* part_off, cudaStream_t s);
// out (accumulated: lanes zeroed, mm[0..cap) = ~0 and mm[cap..2 cap) = 0 by the caller):
// lanes[p*9..] (n, S1 limbs, S2 limbs), mm (min, max), ab[p*4..] = value interval [a, b) and this
// rank's superset range [ia, ib) in the bucketed values
void launch_part_stats(const SegDev* segs, u32 nseg, u32 G, const double* gtab, const u32* off,
                       const u64* T, u32 tstride, const u32* nt, const u32* part_off, u32 cap,
                       const u64* vals, u32 vshift, u32* items /* [cap + 1] */, void* scan_temp,
                       u64* lanes, u64* mm, u64* ab, cudaStream_t s);
#define PART_REC (MOM_LANES + 5)
#define PART_GUESS 16   // part slots per open segment before the exact count is known (a round
                        // with more parts redoes its part moments once with the exact count)
// out[0] = parts, out[1 + p * PART_REC ..] = {lanes[9], min, max, ia, ib, final} (p < cap; final =
// lo == hi or CoV < tp / tq, exact),
// out[1 + cap * PART_REC + s] = nt[s] | kind[s] << 32 (ntk = [nt | kind]); mapped host memory
void launch_part_pack(const u32* part_off, u32 nseg, u32 cap, const u64* lanes, const u64* mm,
                      const u64* ab, const u32* ntk, u32 tp, u32 tq, u64* out, cudaStream_t s);
// ---------------- pass B: assignment + per-(stratum, CTA) statistics -------------------
struct KTab {      // per kernel
  u32 base;        // global id of its first stratum
  u32 m;           // number of strata
  u32 lows_off;    // offset of its strata lower bounds in `lows` (Tier-3 only)
  u32 pad;
};
struct GHash {     // global (sid, cta) table
  u64* keys;       // EMPTY = ~0
  u64* cnt;
  u64* first;
  u64 cap;         // power of two
};
#define HASH_EMPTY 0xFFFFFFFFFFFFFFFFull
int assign_grid();
void launch_assign(const u32* kid, const u64* x, const u32* cta, u64 n, u64 first_id,
                   const KTab* ktab, const u64* lows, u32 K, u32 nlows, u32 ns, u32* sid_out, GHash gh,
                   u64* errflags, int grid, cudaStream_t s);
// compact occupied entries into (key, cnt, first) arrays; *count (device) += entries
void launch_hash_compact(GHash gh, u64* okey, u64* ocnt, u64* ofirst, unsigned long long* count,
                         cudaStream_t s);
void launch_entry_sids(const u64* key, u64 n, u32 ns, u64* out, cudaStream_t s);
void launch_gather_u64(const u64* src, const u32* idx, u64 n, u64* dst, cudaStream_t s);
void launch_iota_u32(u32* p, u64 n, cudaStream_t s);
// reduce duplicates of equal keys (sorted) and pick each stratum's representative
void launch_reps(const u64* key, const u64* cnt, const u64* first, u64 E, const u32* tier,
                 u32 nstrata, u64* rep_id, u64* rep_cta, cudaStream_t s);
// representative (x, y) from the owner rank: out[s] = x, out[nstrata + s] = y (0 if not local)
void launch_rep_xy(const u64* rep_id, u32 nstrata, u64 first_id, u64 n_local, const u64* x,
                   const u64* y, u64* out, cudaStream_t s);

// ---------------- prediction ----------------------------------------------
// strata: W (lo,hi), rep x, rep y ; out[0] = C_pred, out[1] = sum y_rep, out[2] = I (double),
// out[3] = IPC
// ry: [M][nstrata] (one cycle vector per architecture); out: [M][4]
void launch_predict(const u64* W, const u64* rx, const u64* ry, u32 nstrata, u32 M, double* out,
                    cudaStream_t s);

// ---------------- within-stratum cycle moments (Fig. 4 diagnostic) ----------------------------
struct GMomPartial { u64 n, s1lo, s1hi, s2lo, s2hi; };
#define GM_LANES 11   // n, S1 (4 limbs), S2 (6 limbs)
size_t group_moments_part_bytes(u32 nstrata);
// lanes: [nstrata][GM_LANES]; errflag set to 1 if a cycle count >= 2^48 is seen
void launch_group_moments(const u32* sid, const u64* y, u64 n, u32 nstrata, GMomPartial* part,
                          u64* lanes, u64* errflag, cudaStream_t s);

// ---------------- CSV profile ingest (NEXT-4) ---------------------------------------------------
struct CsvSpec { int col_kernel, col_instr, col_cta, col_cycles; int delim; };
u64 csv_tiles(u64 nbytes);
// tile_count: [tiles + 1]; after the first launch tile_count[tiles] = number of '\n'
void launch_csv_count(const unsigned char* buf, u64 nbytes, u32* tile_count, void* scan_temp,
                      cudaStream_t s);
void launch_csv_ends(const unsigned char* buf, u64 nbytes, const u32* tile_off, u64* ends,
                     cudaStream_t s);
void launch_csv_parse(const unsigned char* buf, u64 nbytes, const u64* ends, u64 nends,
                      u64 first_line, u64 nrows, CsvSpec spec, u64* hash, u32* row, u64* name_pos,
                      u64* x, u32* cta, u64* y, u64* errflag, cudaStream_t s);
void launch_csv_heads(const u64* h, u64 n, u32* flag, cudaStream_t s);
void launch_csv_firsts(const u32* flag, const u32* seg, const u32* row, u64 n, u64* first_key,
                       u32* first_val, cudaStream_t s);
void launch_csv_ids(const u32* order, u64 nd, u32* id_of, const u32* flag, const u32* seg,
                    const u32* row, u64 n, u32* kid, cudaStream_t s);
void launch_gather_pairs(const u64* src, const u64* idx, u64 n, u64* dst, cudaStream_t s);
// names of the distinct kernels: text[pos[2d], +pos[2d+1]) -> out[off[d] ...]
void launch_csv_names(const unsigned char* buf, const u64* pos, const u64* off, u64 nd, unsigned char* out,
                      cudaStream_t s);

// ---------------- exact min-strata DP (NEXT-3) --------------------------------------------------
void launch_rle(const u64* keys, const u32* flag, const u32* seg, u64 n, u32 bx, u64* ukey,
                u32* ustart, u32* kstart, cudaStream_t s);
// the min-strata DP by layers (dp.cu): prefix sums and L_0, then per layer k one k_dp_layer and one
// k_dp_compact (lists ping-pong; *remaining = kernels still without f(m))
void launch_dp_prefix(const u64* ukey, const u32* ustart, const u32* kstart, u32 nk, u64 xmask, u32 p, u32 q,
                      u32 max_distinct, u64* Pn, u128* P1, u128* P2, u32* f, u32* count, u32* list,
                      u32* lcnt, u32* state, cudaStream_t s);
void launch_dp_layer(const u32* kstart, u32 nk, u32 nu, u32 k, u32 p, u32 q, const u64* Pn, const u128* P1,
                     const u128* P2, u32* f, u32* arg, const u32* lprev, const u32* lcnt, const u32* state,
                     cudaStream_t s);
void launch_dp_compact(const u32* kstart, u32 nk, u32 k, const u32* f, const u32* arg, const u64* ukey,
                       u64 xmask, u32* lnext, u32* lcnt, u32* state, u32* count, u64* cuts, u32* remaining,
                       cudaStream_t s);
void launch_dp_gather(const u32* kstart, const u32* count, const u64* off, const u64* cuts, u32 nk,
                      u64* out, cudaStream_t s);

// ---------------- misc -------------------------------------------------------------------------
void launch_fill_u64(u64* p, u64 n, u64 v, cudaStream_t s);
#define FILL_MAX 4
struct FillRegions { u64* p[FILL_MAX]; u64 n[FILL_MAX]; u64 v[FILL_MAX]; int k; };
void launch_fill_multi(const FillRegions& r, cudaStream_t s);
// SM-driven copy (device or pinned host memory on either side; no copy engine)
void launch_copy(void* dst, const void* src, u64 bytes, cudaStream_t s);
#define COPY_MAX 8
struct CopyRegions { void* dst[COPY_MAX]; const void* src[COPY_MAX]; u64 bytes[COPY_MAX]; int k; };
void launch_copy_multi(const CopyRegions& r, cudaStream_t s);
// dst[i] = src[i] for a u16 column (SIEVE_KID16 / SIEVE_CTA16 loads)
void launch_widen_u16(const void* src, u64 n, u32* dst, cudaStream_t s);
// cross-rank encoding of u128 pairs [n][2] <-> 4 limbs [n][4]
void launch_u128_to_limbs(const u64* src, u64 n, u64* limbs, cudaStream_t s);
void launch_limbs_to_u128(const u64* limbs, u64 n, u64* dst, cudaStream_t s);
// p[i * stride] = ~p[i * stride], i < n (a MIN all-reduce becomes a MAX on complemented lanes)
void launch_complement(u64* p, u64 n, u64 stride, cudaStream_t s);
// x[0] = (flag[0] != 0), x[1 + r] = (r == rank ? count[0] : 0), r < world
void launch_exchange_prep(const u64* flag, const unsigned long long* count, int rank, int world, u64* x,
                          cudaStream_t s);
