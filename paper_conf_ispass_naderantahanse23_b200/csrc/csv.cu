// csv.cu -- profile ingest (the profiler's per-invocation table "converted
// into a readable CSV file which serves as input"): parse a CSV export
// (Nsight Compute / NVBit style: one row per kernel invocation in launch order, quoted fields
// may contain the delimiter, numbers may carry thousands separators) on the GPU and intern the
// kernel names into dense ids in order of first appearance.
//
//   1. line ends: per-tile newline counts -> exclusive scan -> per-tile positions (2 passes);
//   2. one thread per line: walk the fields (quote-aware), hash the kernel-name field (64-bit
//      FNV-1a over the unquoted bytes), parse the numeric fields;
//   3. interning: radix-sort (hash, row) pairs (stable), mark the first row of every distinct
//      hash, radix-sort the distinct hashes by that first row -> dense ids in first-appearance
//      order, scatter the id back to every row.
// Newlines inside quoted fields are not supported (profiler exports never contain them).
#include "kernels.cuh"

#define CSV_THREADS 256
#define CSV_TB 64   // bytes per thread per tile
#define CSV_TILE (CSV_THREADS * CSV_TB)

void scan_u32(const u32* in, u32* out, u64 n, void* temp, u32* total, cudaStream_t s);

__global__ void __launch_bounds__(CSV_THREADS)
k_csv_count(const unsigned char* __restrict__ buf, u64 nbytes, u32* __restrict__ tile_count) {
  pdl_begin();
  u64 base = (u64)blockIdx.x * CSV_TILE + (u64)threadIdx.x * CSV_TB;
  u32 c = 0;
  for (u32 j = 0; j < CSV_TB; j++) {
    u64 i = base + j;
    if (i < nbytes && buf[i] == '\n') c++;
  }
  for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
  __shared__ u32 s[CSV_THREADS / 32];
  if (lane_id() == 0) s[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    u32 t = 0;
    for (int w = 0; w < CSV_THREADS / 32; w++) t += s[w];
    tile_count[blockIdx.x] = t;
  }
}

// writes the position of every '\n' (line end) in file order
__global__ void __launch_bounds__(CSV_THREADS)
k_csv_ends(const unsigned char* __restrict__ buf, u64 nbytes, const u32* __restrict__ tile_off,
           u64* __restrict__ ends) {
  pdl_begin();
  u64 base = (u64)blockIdx.x * CSV_TILE + (u64)threadIdx.x * CSV_TB;
  u32 c = 0;
  for (u32 j = 0; j < CSV_TB; j++) {
    u64 i = base + j;
    if (i < nbytes && buf[i] == '\n') c++;
  }
  // exclusive prefix of the per-thread counts inside the tile
  u32 inc = c;
  for (int o = 1; o < 32; o <<= 1) {
    u32 v = __shfl_up_sync(0xffffffffu, inc, o);
    if ((int)lane_id() >= o) inc += v;
  }
  __shared__ u32 s[CSV_THREADS / 32];
  if (lane_id() == 31) s[threadIdx.x >> 5] = inc;
  __syncthreads();
  u32 wbase = 0;
  for (u32 w = 0; w < (threadIdx.x >> 5); w++) wbase += s[w];
  u64 o = (u64)tile_off[blockIdx.x] + wbase + inc - c;
  for (u32 j = 0; j < CSV_TB; j++) {
    u64 i = base + j;
    if (i < nbytes && buf[i] == '\n') ends[o++] = i;
  }
}

__device__ __forceinline__ bool parse_u64(const unsigned char* p, u32 len, u64* out) {
  u64 v = 0;
  bool any = false;
  for (u32 i = 0; i < len; i++) {
    unsigned char ch = p[i];
    if (ch >= '0' && ch <= '9') {
      const u64 q = ~0ull / 10;  // 1844674407370955161: v * 10 + d fits iff v < q or v == q, d <= 5
      if (v > q || (v == q && (u32)(ch - '0') > (u32)(~0ull % 10))) return false;
      v = v * 10 + (ch - '0');
      any = true;
    } else if (ch == ',' || ch == '"' || ch == ' ' || ch == '_' || ch == '\r' || ch == '\t') {
      continue;  // thousands separators, quotes, padding
    } else {
      return false;
    }
  }
  *out = v;
  return any;
}

// one thread per data line: fields by a quote-aware walk
__global__ void k_csv_parse(const unsigned char* __restrict__ buf, u64 nbytes,
                            const u64* __restrict__ ends, u64 nends, u64 first_line, u64 nrows,
                            CsvSpec spec, u64* __restrict__ hash, u32* __restrict__ row,
                            u64* __restrict__ name_pos, u64* __restrict__ x, u32* __restrict__ cta,
                            u64* __restrict__ y, u64* errflag) {
  pdl_begin();
  u64 r = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= nrows) return;
  u64 line = first_line + r;
  u64 b = line == 0 ? 0 : ends[line - 1] + 1;
  u64 e = line < nends ? ends[line] : nbytes;
  if (e > b && buf[e - 1] == '\r') e--;
  int field = 0;
  bool inq = false;
  u64 fs = b;
  u64 h = 0xcbf29ce484222325ull;
  u64 vx = 0, vy = 0, vc = 0;
  bool okx = spec.col_instr < 0, oky = spec.col_cycles < 0, okc = spec.col_cta < 0, okn = false;
  u64 npos = 0, nlen = 0;
  for (u64 i = b; i <= e; i++) {
    unsigned char ch = i < e ? buf[i] : (unsigned char)spec.delim;
    if (i < e && ch == '"') { inq = !inq; continue; }
    if (i < e && (inq || ch != (unsigned char)spec.delim)) {
      if (field == spec.col_kernel) { h = (h ^ ch) * 0x100000001b3ull; if (!nlen) npos = i; nlen = i - npos + 1; }
      continue;
    }
    // end of field [fs, i)
    u32 len = (u32)(i - fs);
    if (field == spec.col_kernel) okn = true;
    if (field == spec.col_instr) okx = parse_u64(buf + fs, len, &vx);
    if (field == spec.col_cycles) oky = parse_u64(buf + fs, len, &vy);
    if (field == spec.col_cta) { okc = parse_u64(buf + fs, len, &vc) && vc <= 0xFFFFFFFFull; }
    field++;
    fs = i + 1;
  }
  if (!(okx && oky && okc && okn)) atomicMax((unsigned long long*)errflag, 1ull);
  hash[r] = h;
  row[r] = (u32)r;
  name_pos[2 * r] = npos;
  name_pos[2 * r + 1] = nlen;
  x[r] = vx;
  if (cta) cta[r] = (u32)vc;
  if (y) y[r] = vy;
}

// after sorting (hash, row) by hash (stable): flag[i] = 1 if i starts a new distinct hash
__global__ void k_csv_heads(const u64* __restrict__ h, u64 n, u32* __restrict__ flag) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) flag[i] = (i == 0 || h[i] != h[i - 1]) ? 1u : 0u;
}

// distinct hash d (= exclusive scan of flags at its head): its first row, as a sort key
__global__ void k_csv_firsts(const u32* __restrict__ flag, const u32* __restrict__ seg,
                             const u32* __restrict__ row, u64 n, u64* __restrict__ first_key,
                             u32* __restrict__ first_val) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n && flag[i]) {
    first_key[seg[i]] = row[i];
    first_val[seg[i]] = seg[i];
  }
}

// id of distinct hash d = rank of its first row; scatter to every row
__global__ void k_csv_rank(const u32* __restrict__ order, u64 nd, u32* __restrict__ id_of) {
  pdl_begin();
  u64 r = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (r < nd) id_of[order[r]] = (u32)r;
}
// element i of the hash-sorted list belongs to distinct hash d = (heads up to and incl. i) - 1
__global__ void k_csv_scatter(const u32* __restrict__ flag, const u32* __restrict__ seg,
                              const u32* __restrict__ row, const u32* __restrict__ id_of, u64 n,
                              u32* __restrict__ kid) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) kid[row[i]] = id_of[seg[i] + flag[i] - 1];
}

__global__ void k_gather_pairs(const u64* src, const u64* idx, u64 n, u64* dst) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) { dst[2 * i] = src[2 * idx[i]]; dst[2 * i + 1] = src[2 * idx[i] + 1]; }
}
void launch_gather_pairs(const u64* src, const u64* idx, u64 n, u64* dst, cudaStream_t s) {
  if (n) SV_LAUNCH(k_gather_pairs, div_up(n, 256), 256, 0, s)(src, idx, n, dst);
}

u64 csv_tiles(u64 nbytes) { return (nbytes + CSV_TILE - 1) / CSV_TILE; }

void launch_csv_count(const unsigned char* buf, u64 nbytes, u32* tile_count, void* scan_temp,
                      cudaStream_t s) {
  u64 nt = csv_tiles(nbytes);
  if (!nt) return;
  SV_LAUNCH(k_csv_count, (unsigned)nt, CSV_THREADS, 0, s)(buf, nbytes, tile_count);
  scan_u32(tile_count, tile_count, nt, scan_temp, tile_count + nt, s);
}

void launch_csv_ends(const unsigned char* buf, u64 nbytes, const u32* tile_off, u64* ends,
                     cudaStream_t s) {
  u64 nt = csv_tiles(nbytes);
  if (nt) SV_LAUNCH(k_csv_ends, (unsigned)nt, CSV_THREADS, 0, s)(buf, nbytes, tile_off, ends);
}

void launch_csv_parse(const unsigned char* buf, u64 nbytes, const u64* ends, u64 nends,
                      u64 first_line, u64 nrows, CsvSpec spec, u64* hash, u32* row, u64* name_pos,
                      u64* x, u32* cta, u64* y, u64* errflag, cudaStream_t s) {
  if (nrows)
    SV_LAUNCH(k_csv_parse, div_up(nrows, 128), 128, 0, s)(buf, nbytes, ends, nends, first_line, nrows,
                                                       spec, hash, row, name_pos, x, cta, y, errflag);
}

void launch_csv_heads(const u64* h, u64 n, u32* flag, cudaStream_t s) {
  if (n) SV_LAUNCH(k_csv_heads, div_up(n, 256), 256, 0, s)(h, n, flag);
}
void launch_csv_firsts(const u32* flag, const u32* seg, const u32* row, u64 n, u64* first_key,
                       u32* first_val, cudaStream_t s) {
  if (n) SV_LAUNCH(k_csv_firsts, div_up(n, 256), 256, 0, s)(flag, seg, row, n, first_key, first_val);
}
void launch_csv_ids(const u32* order, u64 nd, u32* id_of, const u32* flag, const u32* seg,
                    const u32* row, u64 n, u32* kid, cudaStream_t s) {
  if (nd) SV_LAUNCH(k_csv_rank, div_up(nd, 256), 256, 0, s)(order, nd, id_of);
  if (n) SV_LAUNCH(k_csv_scatter, div_up(n, 256), 256, 0, s)(flag, seg, row, id_of, n, kid);
}
