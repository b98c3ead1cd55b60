// dp.cu -- exact minimum number of strata ("(1) minimises
// the number of strata such that (2) the CoV of each stratum is below theta"; A28).
//
// Per Tier-3 kernel, over its distinct instruction counts (run-length encoded from the sorted
// Tier-3 keys): f(0) = 0, f(j) = min { f(i) + 1 : CoV(values i+1..j) < theta }, ties -> the
// smallest i; the backtrack from m gives the canonical optimal cuts.  Each (i, j) test is the
// exact u256 comparison q^2 (n S2 - S1^2) < p^2 S1^2 on prefix sums of (count, count*v,
// count*v^2), decided in fp64 when the ratio is further than 1e-12 (relative) from the boundary
// -- far beyond the fp64 error of the ratio (< 8 ulp), so the decision is always the exact one.
//
// B200 mapping: the DP is evaluated by layers, not by j.  Layer k assigns f(j) = k to every j
// not yet assigned that has a valid run (i, j] from some i of layer k-1 (L_{k-1}), with arg(j) =
// the smallest such i: by induction exactly the DP's values and tie rule.  A layer is one launch
// over every kernel's j at once (one thread per j scanning L_{k-1} in ascending order, the
// lanes of a warp sharing the list), then one block per kernel compacts L_k; the layers stop
// when every kernel's f(m) is known.  (Round 1 ran the DP by j in one block per kernel, a
// block-wide minimum per j: 2.0 s for C3's largest kernels against all of the GPU here.)
#include "kernels.cuh"

#define DP_THREADS 1024

struct U256 { u64 w[4]; };

__device__ __forceinline__ U256 mul128(u128 a, u128 b) {
  u64 a0 = (u64)a, a1 = (u64)(a >> 64), b0 = (u64)b, b1 = (u64)(b >> 64);
  u128 p00 = (u128)a0 * b0, p01 = (u128)a0 * b1, p10 = (u128)a1 * b0, p11 = (u128)a1 * b1;
  U256 r;
  r.w[0] = (u64)p00;
  u128 mid = (p00 >> 64) + (u64)p01 + (u64)p10;
  r.w[1] = (u64)mid;
  u128 hi = (mid >> 64) + (p01 >> 64) + (p10 >> 64) + p11;
  r.w[2] = (u64)hi;
  r.w[3] = (u64)(hi >> 64);
  return r;
}
__device__ __forceinline__ U256 mul_u64(U256 a, u64 m) {
  U256 r;
  u128 c = 0;
#pragma unroll
  for (int i = 0; i < 4; i++) {
    u128 t = (u128)a.w[i] * m + c;
    r.w[i] = (u64)t;
    c = t >> 64;
  }
  return r;
}
__device__ __forceinline__ U256 sub256(U256 a, U256 b) {
  U256 r;
  u64 br = 0;
#pragma unroll
  for (int i = 0; i < 4; i++) {
    u64 t = a.w[i] - b.w[i];
    u64 b1 = a.w[i] < b.w[i];
    r.w[i] = t - br;
    br = b1 | (t < br);
  }
  return r;
}
__device__ __forceinline__ bool lt256(U256 a, U256 b) {
#pragma unroll
  for (int i = 3; i >= 0; i--)
    if (a.w[i] != b.w[i]) return a.w[i] < b.w[i];
  return false;
}
__device__ __forceinline__ double to_d(u128 v) {
  return fma((double)(u64)(v >> 64), 18446744073709551616.0, (double)(u64)v);
}

// CoV < p/q of a run with n values, sums s1, s2 (exact decision; fp64 fast path)
__device__ __forceinline__ bool run_ok(u64 n, u128 s1, u128 s2, u32 p, u32 q, double bound) {
  double d1 = to_d(s1);
  double r = ((double)n * to_d(s2)) / (d1 * d1);  // = 1 + CoV^2
  if (r < bound * (1.0 - 1e-12)) return true;
  if (r > bound * (1.0 + 1e-12)) return false;
  U256 nS2 = mul128((u128)n, s2);
  U256 sq = mul128(s1, s1);
  U256 lhs = mul_u64(sub256(nS2, sq), (u64)q * q);
  U256 rhs = mul_u64(sq, (u64)p * p);
  return lt256(lhs, rhs);
}

#define DP_INF 0xFFFFFFFFu

// per Tier-3 rank r: distinct values ukey[kstart[r] .. kstart[r+1]), run starts ustart[] (with
// ustart[nu] = nkeys).  Arrays indexed at off = kstart[r] + r hold m + 1 entries per kernel:
// prefix sums, f, arg and the layer lists.  state[r] = 1 while the kernel's f(m) is unknown.
__global__ void __launch_bounds__(DP_THREADS)
k_dp_prefix(const u64* __restrict__ ukey, const u32* __restrict__ ustart, const u32* __restrict__ kstart,
            u64 xmask, u32 p, u32 q, u32 max_distinct, u64* __restrict__ Pn, u128* __restrict__ P1,
            u128* __restrict__ P2, u32* __restrict__ f, u32* __restrict__ count, u32* __restrict__ list,
            u32* __restrict__ lcnt, u32* __restrict__ state) {
  pdl_begin();
  __shared__ u64 s_n[DP_THREADS];
  __shared__ u128 s_1[DP_THREADS], s_2[DP_THREADS];
  const u32 r = blockIdx.x;
  const u32 b = kstart[r], m = kstart[r + 1] - b;
  const u64 off = (u64)b + r;
  const double bound = 1.0 + ((double)p * p) / ((double)q * q);
  // prefix sums: thread t owns a contiguous chunk
  const u32 T = DP_THREADS, t = threadIdx.x;
  const u32 chunk = (m + T - 1) / T;
  const u32 c0 = min(m, t * chunk), c1 = min(m, c0 + chunk);
  u64 ln = 0;
  u128 l1 = 0, l2 = 0;
  for (u32 i = c0; i < c1; i++) {
    u64 v = ukey[b + i] & xmask, c = ustart[b + i + 1] - ustart[b + i];
    ln += c;
    l1 += (u128)c * v;
    l2 += (u128)c * ((u128)v * v);
  }
  s_n[t] = ln; s_1[t] = l1; s_2[t] = l2;
  __syncthreads();
  if (t == 0) {
    u64 an = 0;
    u128 a1 = 0, a2 = 0;
    for (u32 w = 0; w < T; w++) {
      u64 xn = s_n[w]; u128 x1 = s_1[w], x2 = s_2[w];
      s_n[w] = an; s_1[w] = a1; s_2[w] = a2;
      an += xn; a1 += x1; a2 += x2;
    }
  }
  __syncthreads();
  ln = s_n[t]; l1 = s_1[t]; l2 = s_2[t];
  for (u32 i = c0; i < c1; i++) {
    Pn[off + i] = ln; P1[off + i] = l1; P2[off + i] = l2;
    u64 v = ukey[b + i] & xmask, c = ustart[b + i + 1] - ustart[b + i];
    ln += c;
    l1 += (u128)c * v;
    l2 += (u128)c * ((u128)v * v);
  }
  if (c1 == m && (c0 < c1 || t == 0)) { Pn[off + m] = ln; P1[off + m] = l1; P2[off + m] = l2; }
  for (u32 j = t; j <= m; j += T) f[off + j] = j == 0 ? 0u : DP_INF;
  __syncthreads();
  if (t != 0) return;
  if (run_ok(Pn[off + m], P1[off + m], P2[off + m], p, q, bound)) {   // one stratum
    count[r] = 1;
    state[r] = 0;
  } else if (m > max_distinct) {
    count[r] = 0xFFFFFFFFu;
    state[r] = 0;
  } else {
    list[off] = 0;   // L_0 = {0}
    lcnt[r] = 1;
    state[r] = 1;
  }
}

// layer k: every unassigned j of a live kernel scans L_{k-1} (ascending) for its first valid run
__global__ void k_dp_layer(const u32* __restrict__ kstart, u32 nk, u32 nu, u32 k, u32 p, u32 q,
                           const u64* __restrict__ Pn, const u128* __restrict__ P1,
                           const u128* __restrict__ P2, u32* __restrict__ f, u32* __restrict__ arg,
                           const u32* __restrict__ lprev, const u32* __restrict__ lcnt,
                           const u32* __restrict__ state) {
  pdl_begin();
  const double bound = 1.0 + ((double)p * p) / ((double)q * q);
  for (u32 e = blockIdx.x * blockDim.x + threadIdx.x; e < nu; e += gridDim.x * blockDim.x) {
    u32 lo = 0, hi = nk - 1;   // kernel of distinct value e: last r with kstart[r] <= e
    while (lo < hi) {
      const u32 mid = (lo + hi + 1) >> 1;
      if (kstart[mid] <= e) lo = mid; else hi = mid - 1;
    }
    const u32 r = lo;
    if (!state[r]) continue;
    const u64 off = (u64)kstart[r] + r;
    const u32 j = e - kstart[r] + 1;
    if (f[off + j] != DP_INF) continue;
    const u64 nj = Pn[off + j];
    const u128 sj1 = P1[off + j], sj2 = P2[off + j];
    const u32 cnt = lcnt[r];
    for (u32 x = 0; x < cnt; x++) {
      const u32 i = lprev[off + x];
      if (i >= j) break;
      if (run_ok(nj - Pn[off + i], sj1 - P1[off + i], sj2 - P2[off + i], p, q, bound)) {
        f[off + j] = k;
        arg[off + j] = i;
        break;
      }
    }
  }
}

// one block per live kernel: L_k = { j : f(j) = k } in ascending order; a kernel whose f(m) is
// known is done (its count and canonical cuts written), else it counts into *remaining
__global__ void __launch_bounds__(DP_THREADS)
k_dp_compact(const u32* __restrict__ kstart, u32 k, const u32* __restrict__ f, const u32* __restrict__ arg,
             const u64* __restrict__ ukey, u64 xmask, u32* __restrict__ lnext, u32* __restrict__ lcnt,
             u32* __restrict__ state, u32* __restrict__ count, u64* __restrict__ cuts,
             u32* __restrict__ remaining) {
  pdl_begin();
  __shared__ u32 s_c[DP_THREADS];
  const u32 r = blockIdx.x;
  if (!state[r]) return;
  const u32 b = kstart[r], m = kstart[r + 1] - b;
  const u64 off = (u64)b + r;
  const u32 T = DP_THREADS, t = threadIdx.x;
  const u32 chunk = (m + 1 + T - 1) / T;
  const u32 c0 = min(m + 1, t * chunk), c1 = min(m + 1, c0 + chunk);
  u32 c = 0;
  for (u32 j = c0; j < c1; j++) c += f[off + j] == k;
  s_c[t] = c;
  __syncthreads();
  if (t == 0) {
    u32 a = 0;
    for (u32 w = 0; w < T; w++) { const u32 x = s_c[w]; s_c[w] = a; a += x; }
    lcnt[r] = a;
  }
  __syncthreads();
  u32 o = s_c[t];
  for (u32 j = c0; j < c1; j++)
    if (f[off + j] == k) lnext[off + o++] = j;
  if (t != 0) return;
  const u32 fm = f[off + m];
  if (fm == DP_INF) { atomicAdd(remaining, 1u); return; }
  state[r] = 0;
  count[r] = fm;
  // cuts (lowest value of every stratum but the first), ascending, at cuts[b .. b + fm - 1)
  u32 j = m, w = fm - 1;
  while (j > 0) {
    const u32 i = arg[off + j];
    if (i > 0) cuts[b + (--w)] = ukey[b + i] & xmask;
    j = i;
  }
}

// run heads of sorted keys -> unique keys, run starts (ustart[nu] = n), Tier-3 rank starts
__global__ void k_rle(const u64* __restrict__ keys, const u32* __restrict__ flag,
                      const u32* __restrict__ seg, u64 n, u32 bx, u64* __restrict__ ukey,
                      u32* __restrict__ ustart, u32* __restrict__ kstart) {
  pdl_begin();
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n || !flag[i]) return;
  u32 d = seg[i];
  u64 k = keys[i];
  ukey[d] = k;
  ustart[d] = (u32)i;
  if (i == 0 || (keys[i - 1] >> bx) != (k >> bx)) kstart[k >> bx] = d;
}

__global__ void k_dp_gather(const u32* __restrict__ kstart, const u32* __restrict__ count,
                            const u64* __restrict__ off, const u64* __restrict__ cuts,
                            u64* __restrict__ out) {
  pdl_begin();
  const u32 r = blockIdx.x;
  const u32 c = count[r];
  if (c < 2 || c == 0xFFFFFFFFu) return;
  for (u32 i = threadIdx.x; i + 1 < c; i += blockDim.x) out[off[r] + i] = cuts[kstart[r] + i];
}

void launch_rle(const u64* keys, const u32* flag, const u32* seg, u64 n, u32 bx, u64* ukey,
                u32* ustart, u32* kstart, cudaStream_t s) {
  if (n) SV_LAUNCH(k_rle, div_up(n, 256), 256, 0, s)(keys, flag, seg, n, bx, ukey, ustart, kstart);
}

void launch_dp_prefix(const u64* ukey, const u32* ustart, const u32* kstart, u32 nk, u64 xmask, u32 p, u32 q,
                      u32 max_distinct, u64* Pn, u128* P1, u128* P2, u32* f, u32* count, u32* list,
                      u32* lcnt, u32* state, cudaStream_t s) {
  if (nk)
    SV_LAUNCH(k_dp_prefix, nk, DP_THREADS, 0, s)(ukey, ustart, kstart, xmask, p, q, max_distinct, Pn, P1, P2,
                                                 f, count, list, lcnt, state);
}
void launch_dp_layer(const u32* kstart, u32 nk, u32 nu, u32 k, u32 p, u32 q, const u64* Pn, const u128* P1,
                     const u128* P2, u32* f, u32* arg, const u32* lprev, const u32* lcnt, const u32* state,
                     cudaStream_t s) {
  if (nk && nu)
    SV_LAUNCH(k_dp_layer, min(div_up(nu, 256), (u32)sv_num_sms() * 8), 256, 0, s)(
        kstart, nk, nu, k, p, q, Pn, P1, P2, f, arg, lprev, lcnt, state);
}
void launch_dp_compact(const u32* kstart, u32 nk, u32 k, const u32* f, const u32* arg, const u64* ukey,
                       u64 xmask, u32* lnext, u32* lcnt, u32* state, u32* count, u64* cuts, u32* remaining,
                       cudaStream_t s) {
  if (nk)
    SV_LAUNCH(k_dp_compact, nk, DP_THREADS, 0, s)(kstart, k, f, arg, ukey, xmask, lnext, lcnt, state, count,
                                                  cuts, remaining);
}

void launch_dp_gather(const u32* kstart, const u32* count, const u64* off, const u64* cuts, u32 nk,
                      u64* out, cudaStream_t s) {
  if (nk) SV_LAUNCH(k_dp_gather, nk, 256, 0, s)(kstart, count, off, cuts, out);
}
