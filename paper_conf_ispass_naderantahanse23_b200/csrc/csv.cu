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
#define CSV_TILE (CSV_THREADS * CSV_TB)   // 16 KB: 2 KB per warp

void scan_u32(const u32* in, u32* out, u64 n, void* temp, u32* total, cudaStream_t s);

// newline bytes of a 16-byte chunk as a bit mask (bit i: byte i is '\n'); bytes at or past
// nbytes do not count
__device__ __forceinline__ u32 nl_mask16(const unsigned char* buf, u64 off, u64 nbytes) {
  u32 w[4];
  if (off + 16 <= nbytes && (((uintptr_t)buf + off) & 15) == 0) {
    const uint4 v = __ldg((const uint4*)(buf + off));
    w[0] = v.x; w[1] = v.y; w[2] = v.z; w[3] = v.w;
  } else {
#pragma unroll
    for (int k = 0; k < 4; k++) {
      u32 x = 0;
#pragma unroll
      for (int b = 0; b < 4; b++) {
        const u64 i = off + 4 * k + b;
        x |= (u32)(i < nbytes ? buf[i] : 0) << (8 * b);
      }
      w[k] = x;
    }
  }
  u32 m = 0;
#pragma unroll
  for (int k = 0; k < 4; k++) {
    const u32 e = __vcmpeq4(w[k], 0x0a0a0a0au);   // 0xff in every byte equal to '\n'
    // one bit per byte: bits 7, 15, 23, 31 of e -> bits 4k .. 4k + 3
    const u32 b4 = ((e >> 7) & 1u) | ((e >> 14) & 2u) | ((e >> 21) & 4u) | ((e >> 28) & 8u);
    m |= b4 << (4 * k);
  }
  return m;
}

// A tile of CSV_TILE bytes per block; each warp walks its CSV_TILE / CSV_WARPS bytes as 512-byte
// steps of coalesced 16-byte chunks (one per lane), so the newlines are met in file order.
#define CSV_WARPS (CSV_THREADS / 32)
#define CSV_WBYTES (CSV_TILE / CSV_WARPS)
static_assert(CSV_WBYTES % 512 == 0, "a warp's share of a tile is whole 512-byte steps");

__global__ void __launch_bounds__(CSV_THREADS)
k_csv_count(const unsigned char* __restrict__ buf, u64 nbytes, u32* __restrict__ tile_count) {
  pdl_begin();
  const u64 wbase = (u64)blockIdx.x * CSV_TILE + (u64)(threadIdx.x >> 5) * CSV_WBYTES;
  u32 c = 0;
  for (u32 st = 0; st < CSV_WBYTES; st += 512) {
    const u64 off = wbase + st + 16 * lane_id();
    if (off < nbytes) c += __popc(nl_mask16(buf, off, nbytes));
  }
  for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
  __shared__ u32 s[CSV_WARPS];
  if (lane_id() == 0) s[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    u32 t = 0;
    for (int w = 0; w < CSV_WARPS; w++) t += s[w];
    tile_count[blockIdx.x] = t;
  }
}

// writes the position of every '\n' (line end) in file order
__global__ void __launch_bounds__(CSV_THREADS)
k_csv_ends(const unsigned char* __restrict__ buf, u64 nbytes, const u32* __restrict__ tile_off,
           u64* __restrict__ ends) {
  pdl_begin();
  const u32 warp = threadIdx.x >> 5, lane = lane_id();
  const u64 wbase = (u64)blockIdx.x * CSV_TILE + (u64)warp * CSV_WBYTES;
  // this warp's first output slot: the tile's offset plus the newlines of the warps before it
  u32 c = 0;
  for (u32 st = 0; st < CSV_WBYTES; st += 512) {
    const u64 off = wbase + st + 16 * lane;
    if (off < nbytes) c += __popc(nl_mask16(buf, off, nbytes));
  }
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  __shared__ u32 s[CSV_WARPS];
  if (lane == 0) s[warp] = c;
  __syncthreads();
  u64 o = tile_off[blockIdx.x];
  for (u32 w = 0; w < warp; w++) o += s[w];
  for (u32 st = 0; st < CSV_WBYTES; st += 512) {
    const u64 off = wbase + st + 16 * lane;
    u32 m = off < nbytes ? nl_mask16(buf, off, nbytes) : 0u;
    const u32 k = __popc(m);
    u32 inc = k;   // inclusive prefix over the lanes (file order inside the step)
    for (int d = 1; d < 32; d <<= 1) {
      const u32 v = __shfl_up_sync(0xffffffffu, inc, d);
      if ((int)lane >= d) inc += v;
    }
    u64 q = o + inc - k;
    while (m) {
      const int b = __ffs(m) - 1;
      ends[q++] = off + b;
      m &= m - 1;
    }
    o += __shfl_sync(0xffffffffu, inc, 31);
  }
}

// 64-bit finaliser (murmur3 fmix64): the kernel-name hash mixes eight name bytes at a time
__device__ __forceinline__ u64 fmix64(u64 k) {
  k ^= k >> 33;
  k *= 0xff51afd7ed558ccdull;
  k ^= k >> 33;
  k *= 0xc4ceb9fe1a85ec53ull;
  k ^= k >> 33;
  return k;
}

// One thread per data line, one pass over its bytes: a quote-aware walk that splits the fields,
// hashes the kernel-name field (its unquoted bytes, eight at a time) and accumulates the numeric
// fields as it goes (digits; thousands separators, quotes and padding skipped; anything else, an
// empty field or a value past 2^64 - 1 is an error).  Bytes come from 4-byte word loads (byte
// loads near the buffer's end).  Round 1 read every byte with its own load and re-read each
// numeric field to parse it: 0.66 ms for 2M lines, instruction-bound (ALU 71%, issue 86%).
#define CSV_PT 128                 // lines (threads) per block
__global__ void __launch_bounds__(CSV_PT)
k_csv_parse(const unsigned char* __restrict__ buf, u64 nbytes,
            const u64* __restrict__ ends, u64 nends, u64 first_line, u64 nrows,
            CsvSpec spec, u64* __restrict__ hash, u32* __restrict__ row,
            u64* __restrict__ name_pos, u64* __restrict__ x, u32* __restrict__ cta,
            u64* __restrict__ y, u64* errflag) {
  pdl_begin();
  const u64 r = (u64)blockIdx.x * CSV_PT + threadIdx.x;
  if (r >= nrows) return;
  const bool words = (((uintptr_t)buf) & 3) == 0;
  u64 wa = ~0ull;   // address of the cached word
  u32 w = 0;
  auto at = [&](u64 i) -> u32 {
    const u64 a = i & ~3ull;
    if (words && a + 4 <= nbytes) {
      if (a != wa) { w = __ldg((const unsigned int*)(buf + a)); wa = a; }
      return (w >> (8 * (u32)(i & 3))) & 0xFFu;
    }
    return buf[i];
  };
  const u64 line = first_line + r;
  const u64 b = line == 0 ? 0 : ends[line - 1] + 1;
  u64 e = line < nends ? ends[line] : nbytes;
  if (e > b && at(e - 1) == '\r') e--;
  enum { SKIP = 0, NAME = 1, NX = 2, NC = 3, NY = 4 };
  auto role_of = [&](int f) -> int {
    return f == spec.col_kernel ? NAME : f == spec.col_instr ? NX : f == spec.col_cta ? NC
         : f == spec.col_cycles ? NY : SKIP;
  };
  int field = 0, role = role_of(0);
  bool inq = false;
  u64 h = 0x9e3779b97f4a7c15ull, acc = 0;   // name hash state, pending name bytes
  u32 nb = 0;                               // name bytes
  u64 npos = 0, nlen = 0;
  u64 v = 0;                                // the numeric field being read
  bool any = false, bad = false;
  u64 vx = 0, vy = 0, vc = 0;
  bool okx = spec.col_instr < 0, oky = spec.col_cycles < 0, okc = spec.col_cta < 0, okn = false;
  const u64 q10 = ~0ull / 10;   // v * 10 + d fits iff v < q10, or v == q10 and d <= 5
  for (u64 i = b; i <= e; i++) {
    const u32 ch = i < e ? at(i) : (u32)spec.delim;
    if (i < e && ch == '"') { inq = !inq; continue; }
    if (i < e && (inq || ch != (u32)spec.delim)) {
      if (role == NAME) {
        acc |= (u64)ch << (8 * (nb & 7));
        if ((++nb & 7) == 0) { h = fmix64(h ^ acc); acc = 0; }
        if (!nlen) npos = i;
        nlen = i - npos + 1;
      } else if (role != SKIP) {
        if (ch >= '0' && ch <= '9') {
          const u32 d = ch - '0';
          if (v > q10 || (v == q10 && d > (u32)(~0ull % 10))) bad = true;
          v = v * 10 + d;
          any = true;
        } else if (!(ch == ',' || ch == ' ' || ch == '_' || ch == '\r' || ch == '\t')) {
          bad = true;
        }
      }
      continue;
    }
    // end of field
    if (role == NAME) { okn = true; h = fmix64(h ^ acc ^ ((u64)nb << 56)); }
    else if (role == NX) { okx = any && !bad; vx = v; }
    else if (role == NY) { oky = any && !bad; vy = v; }
    else if (role == NC) { okc = any && !bad && v <= 0xFFFFFFFFull; vc = v; }
    role = role_of(++field);
    v = 0; any = false; bad = false;
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

// the distinct names' bytes, concatenated: name d = text[pos[2d], pos[2d] + pos[2d + 1]) goes to
// out[off[d] ...] (one warp per name; the text may be device-resident)
__global__ void k_csv_names(const unsigned char* __restrict__ buf, const u64* __restrict__ pos,
                            const u64* __restrict__ off, u64 nd, unsigned char* __restrict__ out) {
  pdl_begin();
  const u64 d = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (d >= nd) return;
  const u64 b = pos[2 * d], len = pos[2 * d + 1], o = off[d];
  for (u64 i = lane_id(); i < len; i += 32) out[o + i] = buf[b + i];
}
void launch_csv_names(const unsigned char* buf, const u64* pos, const u64* off, u64 nd, unsigned char* out,
                      cudaStream_t s) {
  if (nd) SV_LAUNCH(k_csv_names, div_up(nd * 32, 256), 256, 0, s)(buf, pos, off, nd, out);
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
    SV_LAUNCH(k_csv_parse, div_up(nrows, CSV_PT), CSV_PT, 0, s)(buf, nbytes, ends, nends, first_line, nrows,
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
