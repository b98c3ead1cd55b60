/*
 * oracle/sieve_oracle.c -- plain, slow, single-threaded CPU oracle for the Sieve
 * stratification back-end (Naderan-Tahan, SeyyedAghaei, Eeckhout, ISPASS'23).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table or constant with the CUDA product path (paper_conf_ispass_naderantahanse23_b200/),
 * and neither side includes the other.
 *
 * Citation form: P:NN = /root/reference/PAPER.md line NN.  Readings A1..A24 and the
 * step names O1..O9 are those of SURVEY.md section 8(c), restated in DESIGN.md section 3.
 *
 * Every function below is written in the order of the paper / the 8(c) reading, with
 * no blocking, fusion or reordering:
 *   O1 group invocations by kernel
 *   O2 exact moments n, S1, S2, lo, hi (u128)
 *   O3 tier: Tier-1 iff lo==hi, Tier-2 iff CoV < theta    P:75-85 (A1-A5)
 *   O4 Tier-1/2: one stratum per kernel
 *   O5 Tier-3 refinement: Gaussian KDE on a grid, valleys, split until CoV < theta
 *                                                         P:89, [8] P:317, [36] P:349 (A6-A15)
 *   O6 stratum numbering by (kernel, lo)                  A23
 *   O7 representative: first-chronological (Tier-1) / first-chronological with the most
 *      dominant CTA size (Tier-2/3)                       P:93, P:103 (A16-A19)
 *   O8 weights W_s = sum of instruction counts
 *   O9 prediction: weighted harmonic-mean IPC, C_pred = I / IPC, error, speedup
 *                                                         P:99-101, P:200-208 (A22)
 *
 * Pins (tests/test_oracle_*.py): tier closed forms and exact-boundary multisets, big-int
 * moments, det_exp vs exp (relative 2^-42), the 2^{-j/256} table vs Python decimal,
 * Q vs e^{-t} 2^40 (<= 1 unit), KDE vs scikit-learn / scipy / direct sums,
 * hand-built valley sequences, symmetric two-point masses, strata invariants,
 * representative brute force, prediction identities (homogeneous cycles => error 0,
 * CPI arithmetic-mean form), an independent Python big-int brute force (oracle/brute.py), and
 * the wide regime (tests/test_oracle_wide.py): u256 -> double vs Python float(int), tiers at
 * n S2 >= 2^128 vs the CoV definition in Fractions, h vs Scott's closed form, D_j >= 2^63, the
 * bisection fallback on a unimodal density.
 *
 * Build: gcc -O2 -std=c11 -ffp-contract=off -fPIC -shared (no -ffast-math: every
 * floating-point step must be the IEEE basic operation written here).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef unsigned __int128 u128;

/* ------------------------------------------------------------------------------------------
 * Status codes (the oracle's own; same numeric meaning as the product's API, re-declared)
 * ------------------------------------------------------------------------------------------ */
#define OR_OK 0
#define OR_EINVAL (-1)
#define OR_ERANGE (-2)
#define OR_ENOMEM (-3)
#define OR_EDOM (-6)
#define OR_ELIMIT (-7)

/* ------------------------------------------------------------------------------------------
 * 256-bit unsigned integers (little-endian 64-bit limbs) for the exact CoV comparison (A5).
 * ------------------------------------------------------------------------------------------ */
typedef struct { uint64_t w[4]; } u256;

static u256 u256_from128(u128 a) {
  u256 r = {{(uint64_t)a, (uint64_t)(a >> 64), 0, 0}};
  return r;
}

/* schoolbook product of two values that each fit in 128 bits; the result fits in 256 */
static u256 u256_mul128(u128 a, u128 b) {
  uint64_t x[2] = {(uint64_t)a, (uint64_t)(a >> 64)};
  uint64_t y[2] = {(uint64_t)b, (uint64_t)(b >> 64)};
  uint64_t r[4] = {0, 0, 0, 0};
  for (int i = 0; i < 2; i++) {
    u128 carry = 0;
    for (int j = 0; j < 2; j++) {
      u128 t = (u128)x[i] * y[j] + r[i + j] + carry;
      r[i + j] = (uint64_t)t;
      carry = t >> 64;
    }
    int k = i + 2;
    while (carry) {
      u128 t = (u128)r[k] + carry;
      r[k] = (uint64_t)t;
      carry = t >> 64;
      k++;
    }
  }
  u256 out = {{r[0], r[1], r[2], r[3]}};
  return out;
}

/* (a * small) where a < 2^256 / small; used for q^2 * (...) and p^2 * (...) */
static u256 u256_mul_u64(u256 a, uint64_t m) {
  u256 r;
  u128 carry = 0;
  for (int i = 0; i < 4; i++) {
    u128 t = (u128)a.w[i] * m + carry;
    r.w[i] = (uint64_t)t;
    carry = t >> 64;
  }
  return r;
}

static u256 u256_sub(u256 a, u256 b) { /* requires a >= b */
  u256 r;
  uint64_t borrow = 0;
  for (int i = 0; i < 4; i++) {
    uint64_t bi = b.w[i] + borrow;
    uint64_t nb = (bi < borrow) || (a.w[i] < bi);
    r.w[i] = a.w[i] - bi;
    borrow = nb;
  }
  return r;
}

static int u256_cmp(u256 a, u256 b) {
  for (int i = 3; i >= 0; i--) {
    if (a.w[i] < b.w[i]) return -1;
    if (a.w[i] > b.w[i]) return 1;
  }
  return 0;
}

/* correctly rounded (round-to-nearest-even) conversion of a 256-bit integer to double */
static double u256_to_double(u256 a) {
  if (a.w[3] == 0 && a.w[2] == 0) {
    u128 v = ((u128)a.w[1] << 64) | a.w[0];
    return (double)v; /* libgcc __floatuntidf: correctly rounded */
  }
  int top = a.w[3] ? 3 : 2;
  int bits = 64 * top + (64 - __builtin_clzll(a.w[top]));
  int s = bits - 64; /* keep the top 64 bits, OR the rest into a sticky LSB */
  uint64_t t = 0, sticky = 0;
  for (int b = 0; b < 64; b++) {
    int src = s + b;
    if ((a.w[src / 64] >> (src % 64)) & 1u) t |= (uint64_t)1 << b;
  }
  for (int b = 0; b < s; b++)
    if ((a.w[b / 64] >> (b % 64)) & 1u) { sticky = 1; break; }
  return ldexp((double)(t | sticky), s); /* >= 11 dropped bits, so the sticky LSB is exact */
}

/* test hook (pinned against Python's correctly rounded float(int)): w = 4 little-endian limbs */
double oracle_u256_to_double(const uint64_t* w) {
  u256 a = {{w[0], w[1], w[2], w[3]}};
  return u256_to_double(a);
}

/* ------------------------------------------------------------------------------------------
 * O3 tier rule.  CoV = sigma/mu with population sigma (A1: "the average
 * squared differences with the mean").  CoV < p/q  <=>  q^2 (n S2 - S1^2) < p^2 S1^2 (A3, A5).
 * Tier-1 iff lo == hi (A4).  CoV exactly theta is Tier-3 (A2, "otherwise").
 * ------------------------------------------------------------------------------------------ */
static int cov_below(uint64_t n, u128 S1, u128 S2, uint32_t p, uint32_t q) {
  u256 nS2 = u256_mul128((u128)n, S2);
  u256 S1sq = u256_mul128(S1, S1);
  u256 diff = u256_sub(nS2, S1sq); /* n S2 - S1^2 >= 0 by Cauchy-Schwarz */
  u256 lhs = u256_mul_u64(diff, (uint64_t)q * q);
  u256 rhs = u256_mul_u64(S1sq, (uint64_t)p * p);
  return u256_cmp(lhs, rhs) < 0;
}

int oracle_tier(uint64_t n, uint64_t s1_lo, uint64_t s1_hi, uint64_t s2_lo, uint64_t s2_hi,
                uint64_t lo, uint64_t hi, uint32_t p, uint32_t q) {
  u128 S1 = ((u128)s1_hi << 64) | s1_lo, S2 = ((u128)s2_hi << 64) | s2_lo;
  if (lo == hi) return 1;
  return cov_below(n, S1, S2, p, q) ? 2 : 3;
}

/* ------------------------------------------------------------------------------------------
 * O5a bandwidth: Scott's normal-reference rule [36] P:349 (A8):
 *   var = rn(n S2 - S1^2) / (rn(n) * rn(n)),  sigma = sqrt(var),
 *   h_raw = (bw_scale * sigma) * pow(n, -0.2),  h = h_raw rounded to 16 significant bits.
 * ------------------------------------------------------------------------------------------ */
double oracle_bandwidth(uint64_t n, uint64_t s1_lo, uint64_t s1_hi, uint64_t s2_lo,
                        uint64_t s2_hi, double bw_scale) {
  u128 S1 = ((u128)s1_hi << 64) | s1_lo, S2 = ((u128)s2_hi << 64) | s2_lo;
  u256 diff = u256_sub(u256_mul128((u128)n, S2), u256_mul128(S1, S1));
  double dn = (double)n;
  double var = u256_to_double(diff) / (dn * dn);
  double sigma = sqrt(var);
  double h_raw = (bw_scale * sigma) * pow(dn, -0.2);
  int e = ilogb(h_raw) - 15;
  return ldexp(rint(ldexp(h_raw, -e)), e);
}

/* O5b grid point j on [lo, hi] inclusive (A9): g_j = rn(lo) + rn((hi-lo)*j) / rn(G-1) */
static double grid_point(uint64_t lo, uint64_t hi, uint32_t j, uint32_t G) {
  double a = (double)lo;
  double b = (double)((hi - lo) * (uint64_t)j);
  double c = (double)(G - 1);
  return a + b / c;
}

double oracle_grid_point(uint64_t lo, uint64_t hi, uint32_t j, uint32_t G) {
  return grid_point(lo, hi, j, G);
}

/* ------------------------------------------------------------------------------------------
 * O5c fixed-point Gaussian kernel value (A10), built only from IEEE basic operations:
 *   k = nearest integer to t * 256 log2 e (one rounding, fma), j = k mod 256, m = k div 256
 *   r = fma(-k, rn(ln2 / 256), t)                                  (|r| <= ln2 / 512 + tiny)
 *   P(r) = 1 - r + r^2/2 - r^3/6                                    (Horner with fma)
 *   e^{-t} = 2^{-j/256} * 2^{-m} * e^{-r}
 *   Q = rint(P * T_j * 2^(40 - m)) with ONE rounding: S = ldexp(T_j, 40 - m) is exact and
 *       Q = fma(P, S, 2^52) - 2^52 (the fma lands in [2^52, 2^53), where the ulp is 1).
 *   T_j = 2^{-j/256} correctly rounded for j >= 1 (pinned in tests against Python's decimal
 *       module), T_0 = 1 - 2^-53: with every T_j having fewer than 12 trailing zero bits in its
 *       significand, P * S can never be an exact half-integer (pinned), so Q does not depend on
 *       a tie rule and a sum of terms may be rounded into an accumulator in any order.
 * Q = 0 for k > 10526 (t > 28.5014): there e^{-t} 2^40 < 0.47 rounds to 0 anyway.
 * Fixed point at 2^-40 of one kernel's peak: the relative accuracy of P T_j (< 2^-42) keeps
 * every Q within one unit of e^{-t} 2^40 (pinned).
 * ------------------------------------------------------------------------------------------ */
static const double OR_LOG2E_256 = 256.0 * 1.4426950408889634074;       /* exact scaling */
static const double OR_LN2_256 = 0x1.62e42fefa39efp-9;                  /* rn(ln 2) / 256 */
static const double OR_TWO52 = 4503599627370496.0;
static const double OR_KMAX = 10526.0;                                  /* rint(28.5 * 256 log2 e) */
static const double OR_EXP2_NEG[256] = {
    0x1.fffffffffffffp-1, /* 1 - 2^-53, not 1: see T_j above */ 0x1.fe9d96b2a23d9p-1, 0x1.fd3c22b8f71f1p-1, 0x1.fbdba3692d514p-1,
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

/* the reduced argument and polynomial shared by det_exp and Q.  k is the integer nearest to
 * t * 256 log2 e with a SINGLE rounding: fma(t, C, 1.5 * 2^52) lands in [2^52, 2^53) where the
 * ulp is 1, and subtracting 1.5 * 2^52 back is exact.  Requires k <= OR_KMAX. */
static double exp_reduce(double t, double k, int* j, int* m) {
  int ki = (int)k;
  *j = ki & 255;
  *m = ki >> 8;
  double r = fma(-k, OR_LN2_256, t);
  double p = -1.0 / 6.0;
  p = fma(p, r, 0.5);
  p = fma(p, r, -1.0);
  p = fma(p, r, 1.0);
  return p;
}
static double exp_k(double t) { return fma(t, OR_LOG2E_256, 6755399441055744.0) - 6755399441055744.0; }

/* e^{-t} for t in [0, 28.5] as the method evaluates it (diagnostic / pin only) */
double oracle_det_exp(double t) {
  int j, m;
  double k = exp_k(t);
  if (k > OR_KMAX) return 0.0;
  double p = exp_reduce(t, k, &j, &m);
  return ldexp(p * OR_EXP2_NEG[j], -m);
}

uint64_t oracle_q(double t) {
  double k = exp_k(t);
  if (!(k <= OR_KMAX)) return 0;   /* also t = inf / nan */
  int j, m;
  double p = exp_reduce(t, k, &j, &m);
  double S = ldexp(OR_EXP2_NEG[j], 40 - m);
  return (uint64_t)(fma(p, S, OR_TWO52) - OR_TWO52);
}

double oracle_exp2_table(int j) { return OR_EXP2_NEG[j & 255]; }

/* fixed-point kernel value Q(x, g) (A10): both points are measured from the segment's lo in
 * units of h, gs = rn(rn(g - rn(lo)) * inv_h) and xs = rn(rn(x - lo) * inv_h) (x - lo is an exact
 * integer), z = gs - xs, t = (z * z) * 0.5 */
static double scaled_value(uint64_t x, uint64_t lo, double inv_h) { return (double)(x - lo) * inv_h; }
static double scaled_grid(double g, uint64_t lo, double inv_h) { return (g - (double)lo) * inv_h; }
static uint64_t kernel_q(double gs, double xs) {
  double z = gs - xs;
  double t = (z * z) * 0.5;
  return oracle_q(t);
}

/* O5c density on the grid: D_j = sum over the segment's values of Q(x, g_j), u128 */
static void kde_grid(const uint64_t* v, uint64_t m, uint64_t lo, uint64_t hi, double h,
                     uint32_t G, u128* D) {
  double inv_h = 1.0 / h;
  for (uint32_t j = 0; j < G; j++) {
    double gs = scaled_grid(grid_point(lo, hi, j, G), lo, inv_h);
    u128 acc = 0;
    for (uint64_t i = 0; i < m; i++) acc += kernel_q(gs, scaled_value(v[i], lo, inv_h));
    D[j] = acc;
  }
}

void oracle_kde(const uint64_t* v, uint64_t m, uint64_t lo, uint64_t hi, double h, uint32_t G,
                uint64_t* d_lo, uint64_t* d_hi) {
  u128* D = (u128*)malloc(sizeof(u128) * G);
  kde_grid(v, m, lo, hi, h, G, D);
  for (uint32_t j = 0; j < G; j++) { d_lo[j] = (uint64_t)D[j]; d_hi[j] = (uint64_t)(D[j] >> 64); }
  free(D);
}

/* ------------------------------------------------------------------------------------------
 * O5d valleys (A11): hysteresis two-state scan with delta = max(1, Dmax >> shift); a cut at
 * the midpoint of the minimum's run; the edges are never valleys.  Returns #cut indices.
 * ------------------------------------------------------------------------------------------ */
static uint32_t valleys(const u128* D, uint32_t G, uint32_t shift, uint32_t* cut_idx) {
  u128 dmax = 0;
  for (uint32_t j = 0; j < G; j++) if (D[j] > dmax) dmax = D[j];
  u128 delta = dmax >> shift;
  if (delta < 1) delta = 1;
  int seek_min = 0;
  u128 mx = D[0], mn = 0;
  uint32_t a = 0, b = 0, nc = 0;
  for (uint32_t j = 1; j < G; j++) {
    u128 d = D[j];
    if (!seek_min) {
      if (d > mx) mx = d;
      if (d + delta <= mx) { seek_min = 1; mn = d; a = b = j; }
    } else {
      if (d < mn) { mn = d; a = b = j; }
      else if (d == mn && b == j - 1) { b = j; }
      else if (d >= mn + delta) { cut_idx[nc++] = (a + b) / 2; seek_min = 0; mx = d; }
    }
  }
  return nc;
}

uint32_t oracle_valleys(const uint64_t* d_lo, const uint64_t* d_hi, uint32_t G, uint32_t shift,
                        uint32_t* cut_idx) {
  u128* D = (u128*)malloc(sizeof(u128) * G);
  for (uint32_t j = 0; j < G; j++) D[j] = ((u128)d_hi[j] << 64) | d_lo[j];
  uint32_t nc = valleys(D, G, shift, cut_idx);
  free(D);
  return nc;
}

/* ------------------------------------------------------------------------------------------
 * Result object
 * ------------------------------------------------------------------------------------------ */
typedef struct {
  uint32_t kernel_id, tier, index_in_kernel, rep_cta;
  uint64_t lo, hi, count, instr_sum_lo, instr_sum_hi;
  uint64_t rep_id, rep_instr, rep_cycles;
  double bandwidth;
  uint32_t split_round, pad;
} oracle_stratum;

typedef struct {
  uint32_t kernel_id, round, split_kind, n_cuts;
  uint64_t lo, hi, count;
  double bandwidth;
  uint64_t *d_lo, *d_hi, *cuts;
} oracle_segment;

typedef struct {
  double predicted_cycles, predicted_ipc, measured_cycles, error, speedup;
  uint64_t total_instr_lo, total_instr_hi;
} oracle_prediction;

typedef struct {
  uint64_t n;
  uint32_t G;
  oracle_stratum* strata;
  uint64_t n_strata;
  uint32_t* sid; /* per input row */
  oracle_segment* segs;
  uint64_t n_segs, cap_segs;
  int has_cycles;
  u128 c_meas;
  u128 total_instr;
  uint32_t rounds;
  uint64_t kde_terms_nonzero;
} oracle_result;

/* a candidate part / open segment of one Tier-3 kernel */
typedef struct {
  uint32_t kid;
  uint64_t* v; /* its instruction counts (owned) */
  uint64_t n;
  u128 S1, S2;
  uint64_t lo, hi;
  double h_from; /* bandwidth of the segment whose split created it */
  uint32_t round_from;
} part_t;

static void moments(const uint64_t* v, uint64_t m, u128* S1, u128* S2, uint64_t* lo,
                    uint64_t* hi) {
  u128 s1 = 0, s2 = 0;
  uint64_t l = UINT64_MAX, h = 0;
  for (uint64_t i = 0; i < m; i++) {
    s1 += v[i];
    s2 += (u128)v[i] * v[i];
    if (v[i] < l) l = v[i];
    if (v[i] > h) h = v[i];
  }
  *S1 = s1; *S2 = s2; *lo = l; *hi = h;
}

typedef struct { uint32_t kid; uint64_t lo, hi, n; u128 S1; uint32_t tier; double h; uint32_t round; } fin_t;

static int push_seg(oracle_result* R, oracle_segment s) {
  if (R->n_segs == R->cap_segs) {
    uint64_t nc = R->cap_segs ? 2 * R->cap_segs : 64;
    oracle_segment* ns = (oracle_segment*)realloc(R->segs, nc * sizeof(oracle_segment));
    if (!ns) return OR_ENOMEM;
    R->segs = ns; R->cap_segs = nc;
  }
  R->segs[R->n_segs++] = s;
  return OR_OK;
}

static int cmp_fin(const void* a, const void* b) {
  const fin_t* x = (const fin_t*)a; const fin_t* y = (const fin_t*)b;
  if (x->kid != y->kid) return x->kid < y->kid ? -1 : 1;
  if (x->lo != y->lo) return x->lo < y->lo ? -1 : 1;
  return 0;
}

void oracle_free(oracle_result* R) {
  if (!R) return;
  for (uint64_t i = 0; i < R->n_segs; i++) {
    free(R->segs[i].d_lo); free(R->segs[i].d_hi); free(R->segs[i].cuts);
  }
  free(R->segs); free(R->strata); free(R->sid); free(R);
}

/* ------------------------------------------------------------------------------------------
 * The whole back-end, O1..O8.
 * ids: global invocation id per row (nullable: row index), used for "first-chronological"
 * (A18) so that a subset of kernels can be stratified with their original ids.
 * ------------------------------------------------------------------------------------------ */
int oracle_stratify(uint64_t n, uint32_t K, const uint32_t* kid, const uint64_t* x,
                    const uint32_t* cta, const uint64_t* cycles, const uint64_t* ids,
                    uint32_t theta_num, uint32_t theta_den, uint32_t G, uint32_t valley_shift,
                    uint32_t max_rounds, double bw_scale, int keep_debug, oracle_result** out) {
  *out = NULL;
  if (theta_num == 0 || theta_den == 0 || G < 3 || G > 65536 || K == 0 || valley_shift > 120)
    return OR_EINVAL;
  for (uint64_t i = 0; i < n; i++) {
    if (kid[i] >= K) return OR_EINVAL;
    if (x[i] == 0 || x[i] >= ((uint64_t)1 << 44)) return OR_ERANGE; /* A21 */
  }
  oracle_result* R = (oracle_result*)calloc(1, sizeof(oracle_result));
  if (!R) return OR_ENOMEM;
  R->n = n; R->G = G; R->has_cycles = cycles != NULL;
  R->sid = (uint32_t*)malloc(sizeof(uint32_t) * (n ? n : 1));

  /* O1 group by kernel id (counting sort, stable in row order) */
  uint64_t* cnt = (uint64_t*)calloc(K + 1, sizeof(uint64_t));
  for (uint64_t i = 0; i < n; i++) cnt[kid[i] + 1]++;
  for (uint32_t k = 0; k < K; k++) cnt[k + 1] += cnt[k];
  uint64_t* rows = (uint64_t*)malloc(sizeof(uint64_t) * (n ? n : 1));
  uint64_t* pos = (uint64_t*)malloc(sizeof(uint64_t) * (K + 1));
  memcpy(pos, cnt, sizeof(uint64_t) * (K + 1));
  for (uint64_t i = 0; i < n; i++) rows[pos[kid[i]]++] = i;
  free(pos);

  fin_t* fin = NULL;
  uint64_t n_fin = 0, cap_fin = 0;
#define PUSH_FIN(F) do { if (n_fin == cap_fin) { cap_fin = cap_fin ? 2 * cap_fin : 256; \
      fin = (fin_t*)realloc(fin, cap_fin * sizeof(fin_t)); } fin[n_fin++] = (F); } while (0)

  int status = OR_OK;
  uint32_t max_round_seen = 0;
  u128* D = (u128*)malloc(sizeof(u128) * G);
  uint32_t* cut_idx = (uint32_t*)malloc(sizeof(uint32_t) * G);
  uint64_t* T = (uint64_t*)malloc(sizeof(uint64_t) * (G + 1));

  for (uint32_t k = 0; k < K && status == OR_OK; k++) {
    uint64_t m = cnt[k + 1] - cnt[k];
    if (m == 0) continue;
    uint64_t* v = (uint64_t*)malloc(sizeof(uint64_t) * m);
    for (uint64_t j = 0; j < m; j++) v[j] = x[rows[cnt[k] + j]];
    /* O2 exact moments */
    u128 S1, S2; uint64_t lo, hi;
    moments(v, m, &S1, &S2, &lo, &hi);
    R->total_instr += S1;
    /* O3 tier */
    uint32_t tier = lo == hi ? 1 : (cov_below(m, S1, S2, theta_num, theta_den) ? 2 : 3);
    if (tier != 3) { /* O4 */
      fin_t f = {k, lo, hi, m, S1, tier, 0.0, 0};
      PUSH_FIN(f);
      free(v);
      continue;
    }
    /* O5 Tier-3 refinement: open <- [(k, all invocations of k)] */
    part_t* open = (part_t*)malloc(sizeof(part_t));
    uint64_t n_open = 1;
    open[0].kid = k; open[0].v = v; open[0].n = m; open[0].S1 = S1; open[0].S2 = S2;
    open[0].lo = lo; open[0].hi = hi;
    uint32_t round = 0;
    while (n_open > 0) {
      round++;
      if (round > max_rounds) { status = OR_ELIMIT; break; }
      if (round > max_round_seen) max_round_seen = round;
      part_t* next = NULL;
      uint64_t n_next = 0, cap_next = 0;
      for (uint64_t s = 0; s < n_open; s++) { /* open segments in (k, lo) order */
        part_t* P = &open[s];
        /* a. bandwidth */
        double h = oracle_bandwidth(P->n, (uint64_t)P->S1, (uint64_t)(P->S1 >> 64),
                                    (uint64_t)P->S2, (uint64_t)(P->S2 >> 64), bw_scale);
        /* b, c. grid and fixed-point density */
        kde_grid(P->v, P->n, P->lo, P->hi, h, G, D);
        /* d. valleys -> thresholds T = ceil(g_m), deduplicated, lo < T <= hi */
        uint32_t nc = valleys(D, G, valley_shift, cut_idx);
        uint32_t nt = 0;
        for (uint32_t c = 0; c < nc; c++) {
          double gm = grid_point(P->lo, P->hi, cut_idx[c], G);
          uint64_t t = (uint64_t)ceil(gm);
          if (t <= P->lo || t > P->hi) continue;
          if (nt > 0 && T[nt - 1] == t) continue;
          T[nt++] = t;
        }
        uint32_t kind = 1;
        /* e. fallback: value-range bisection */
        if (nt == 0) { T[nt++] = (P->lo + P->hi + 1) >> 1; kind = 2; }
        if (keep_debug) {
          oracle_segment sg;
          sg.kernel_id = k; sg.round = round; sg.split_kind = kind; sg.n_cuts = nt;
          sg.lo = P->lo; sg.hi = P->hi; sg.count = P->n; sg.bandwidth = h;
          sg.d_lo = (uint64_t*)malloc(8 * G); sg.d_hi = (uint64_t*)malloc(8 * G);
          sg.cuts = (uint64_t*)malloc(8 * nt);
          for (uint32_t j = 0; j < G; j++) { sg.d_lo[j] = (uint64_t)D[j]; sg.d_hi[j] = (uint64_t)(D[j] >> 64); }
          for (uint32_t c = 0; c < nt; c++) sg.cuts[c] = T[c];
          push_seg(R, sg);
        }
        /* f. parts: x < T1 | T1 <= x < T2 | ... ; empty parts dropped */
        for (uint32_t q = 0; q <= nt; q++) {
          uint64_t a = q == 0 ? 0 : T[q - 1];
          uint64_t b = q == nt ? UINT64_MAX : T[q];
          uint64_t pm = 0;
          for (uint64_t i = 0; i < P->n; i++) if (P->v[i] >= a && P->v[i] < b) pm++;
          if (pm == 0) continue;
          uint64_t* pv = (uint64_t*)malloc(sizeof(uint64_t) * pm);
          uint64_t w = 0;
          for (uint64_t i = 0; i < P->n; i++) if (P->v[i] >= a && P->v[i] < b) pv[w++] = P->v[i];
          part_t np;
          np.kid = k; np.v = pv; np.n = pm;
          moments(pv, pm, &np.S1, &np.S2, &np.lo, &np.hi);
          np.h_from = h; np.round_from = round;
          if (np.lo == np.hi || cov_below(np.n, np.S1, np.S2, theta_num, theta_den)) {
            fin_t f = {k, np.lo, np.hi, np.n, np.S1, 3, h, round};
            PUSH_FIN(f);
            free(pv);
          } else {
            if (n_next == cap_next) { cap_next = cap_next ? 2 * cap_next : 8;
              next = (part_t*)realloc(next, cap_next * sizeof(part_t)); }
            next[n_next++] = np;
          }
        }
      }
      for (uint64_t s = 0; s < n_open; s++) free(open[s].v);
      free(open);
      open = next; n_open = n_next;
      /* next round's open set stays in (k, lo) order: parts were appended by ascending value */
    }
    for (uint64_t s = 0; s < n_open; s++) free(open[s].v);
    free(open);
  }
  free(D); free(cut_idx); free(T);
  R->rounds = max_round_seen;
  if (status != OR_OK) { free(fin); free(rows); free(cnt); oracle_free(R); return status; }

  /* O6 global stratum order by (kid, lo) */
  qsort(fin, n_fin, sizeof(fin_t), cmp_fin);
  R->n_strata = n_fin;
  R->strata = (oracle_stratum*)calloc(n_fin ? n_fin : 1, sizeof(oracle_stratum));
  uint64_t* kbase = (uint64_t*)malloc(sizeof(uint64_t) * (K + 1));
  for (uint32_t k = 0; k <= K; k++) kbase[k] = UINT64_MAX;
  for (uint64_t s = 0; s < n_fin; s++) {
    oracle_stratum* o = &R->strata[s];
    if (kbase[fin[s].kid] == UINT64_MAX) kbase[fin[s].kid] = s;
    o->kernel_id = fin[s].kid; o->tier = fin[s].tier;
    o->index_in_kernel = (uint32_t)(s - kbase[fin[s].kid]);
    o->lo = fin[s].lo; o->hi = fin[s].hi; o->count = fin[s].n;
    o->instr_sum_lo = (uint64_t)fin[s].S1; o->instr_sum_hi = (uint64_t)(fin[s].S1 >> 64);
    o->bandwidth = fin[s].h; o->split_round = fin[s].round;
  }

  /* assignment: each invocation goes to the stratum of its kernel whose [lo, hi] holds x */
  for (uint64_t i = 0; i < n; i++) {
    uint32_t k = kid[i];
    uint64_t s = kbase[k];
    while (!(x[i] >= R->strata[s].lo && x[i] <= R->strata[s].hi)) s++;
    R->sid[i] = (uint32_t)s;
  }

  /* O7 representatives.  Tier-1: first-chronological invocation.  Tier-2/3: per CTA value,
   * (count, first id); dominant = max count, ties to the smaller first id; rep = its first. */
  for (uint64_t s = 0; s < n_fin; s++) {
    oracle_stratum* o = &R->strata[s];
    uint32_t k = o->kernel_id;
    uint64_t m = cnt[k + 1] - cnt[k];
    /* the stratum's members, in row order */
    uint64_t nm = 0;
    uint64_t* mem = (uint64_t*)malloc(sizeof(uint64_t) * m);
    for (uint64_t j = 0; j < m; j++) { uint64_t r = rows[cnt[k] + j]; if (R->sid[r] == s) mem[nm++] = r; }
    uint64_t best_row = mem[0], best_id = ids ? ids[mem[0]] : mem[0];
    for (uint64_t j = 1; j < nm; j++) {
      uint64_t id = ids ? ids[mem[j]] : mem[j];
      if (id < best_id) { best_id = id; best_row = mem[j]; }
    }
    if (o->tier != 1) {
      /* distinct CTA values with count and first id (quadratic, plain) */
      uint32_t* cv = (uint32_t*)malloc(sizeof(uint32_t) * nm);
      uint64_t* cc = (uint64_t*)malloc(sizeof(uint64_t) * nm);
      uint64_t* cf = (uint64_t*)malloc(sizeof(uint64_t) * nm);
      uint64_t* cr = (uint64_t*)malloc(sizeof(uint64_t) * nm);
      uint64_t nd = 0;
      for (uint64_t j = 0; j < nm; j++) {
        uint32_t c = cta ? cta[mem[j]] : 0;
        uint64_t id = ids ? ids[mem[j]] : mem[j];
        uint64_t d = 0;
        while (d < nd && cv[d] != c) d++;
        if (d == nd) { cv[nd] = c; cc[nd] = 0; cf[nd] = id; cr[nd] = mem[j]; nd++; }
        cc[d]++;
        if (id < cf[d]) { cf[d] = id; cr[d] = mem[j]; }
      }
      uint64_t b = 0;
      for (uint64_t d = 1; d < nd; d++)
        if (cc[d] > cc[b] || (cc[d] == cc[b] && cf[d] < cf[b])) b = d;
      best_id = cf[b]; best_row = cr[b];
      free(cv); free(cc); free(cf); free(cr);
    }
    o->rep_id = best_id;
    o->rep_cta = cta ? cta[best_row] : 0;
    o->rep_instr = x[best_row];
    o->rep_cycles = cycles ? cycles[best_row] : 0;
    free(mem);
  }

  /* totals: I = sum of W_s (O8), C_meas = sum of y (O9) */
  if (cycles) { u128 c = 0; for (uint64_t i = 0; i < n; i++) c += cycles[i]; R->c_meas = c; }
  free(kbase); free(fin); free(rows); free(cnt);
  *out = R;
  return OR_OK;
}

/* ------------------------------------------------------------------------------------------
 * O8/O9 prediction:
 *   w_s = W_s / I;  IPC_s = x_rep / y_rep;  IPC = 1 / sum_s w_s / IPC_s;
 *   C_pred = I / IPC = sum_s W_s * y_rep / x_rep  (accumulated in __float128, then rounded);
 *   error = |C_pred - C_meas| / C_meas;  speedup = C_meas / sum_s y_rep.
 * rep_cycles: nullable; else per-stratum cycles of the representatives (e.g. simulated).
 * ------------------------------------------------------------------------------------------ */
int oracle_predict(const oracle_result* R, const uint64_t* rep_cycles, oracle_prediction* out) {
  if (!R->has_cycles && !rep_cycles) return OR_EDOM;
  __float128 cp = 0, yrep = 0, I = 0;
  for (uint64_t s = 0; s < R->n_strata; s++) {
    const oracle_stratum* o = &R->strata[s];
    u128 W = ((u128)o->instr_sum_hi << 64) | o->instr_sum_lo;
    uint64_t y = rep_cycles ? rep_cycles[s] : o->rep_cycles;
    cp += ((__float128)W * (__float128)y) / (__float128)o->rep_instr;
    yrep += (__float128)y;
    I += (__float128)W;
  }
  out->predicted_cycles = (double)cp;
  out->predicted_ipc = (double)(I / cp);
  out->total_instr_lo = (uint64_t)R->total_instr;
  out->total_instr_hi = (uint64_t)(R->total_instr >> 64);
  if (R->has_cycles) {
    __float128 cm = (__float128)R->c_meas;
    out->measured_cycles = (double)cm;
    out->error = R->c_meas == 0 ? NAN : (double)((cp > cm ? cp - cm : cm - cp) / cm);
    out->speedup = (double)(cm / yrep);
  } else {
    out->measured_cycles = NAN; out->error = NAN; out->speedup = NAN;
  }
  return OR_OK;
}

/* ------------------------------------------------------------------------------------------
 * Within-stratum cycle variability (Fig. 4): per stratum, the coefficient of
 * variation of the members' cycle counts, cov_s = sigma_pop(y) / mu(y) = sqrt(n S2 - S1^2) / S1
 * (exact integers, one rounding each for the root argument, the root and the division;
 * 0 if S1 == 0), and the average weighted by the strata's instruction weights w_s = W_s / I
 * (reading A25: the paper says "(weighted) average" without naming the weights; Sieve's own
 * weights are the natural choice).  Cycles must be < 2^48.
 * ------------------------------------------------------------------------------------------ */
int oracle_cycle_cov(const oracle_result* R, const uint64_t* cycles, double* cov, double* weighted) {
  uint64_t ns = R->n_strata;
  uint64_t* cnt = (uint64_t*)calloc(ns ? ns : 1, sizeof(uint64_t));
  u128* s1 = (u128*)calloc(ns ? ns : 1, sizeof(u128));
  u256* s2 = (u256*)calloc(ns ? ns : 1, sizeof(u256));
  for (uint64_t i = 0; i < R->n; i++) {
    uint32_t s = R->sid[i];
    uint64_t y = cycles[i];
    if (y >= ((uint64_t)1 << 48)) { free(cnt); free(s1); free(s2); return OR_ERANGE; }
    cnt[s]++;
    s1[s] += y;
    u256 q = u256_mul128((u128)y, (u128)y);
    u128 lo = ((u128)s2[s].w[1] << 64) | s2[s].w[0];
    u128 sum = lo + (((u128)q.w[1] << 64) | q.w[0]);
    u128 carry = sum < lo ? 1 : 0;
    s2[s].w[0] = (uint64_t)sum; s2[s].w[1] = (uint64_t)(sum >> 64);
    u128 hi = ((u128)s2[s].w[3] << 64) | s2[s].w[2];
    hi += carry + (((u128)q.w[3] << 64) | q.w[2]);
    s2[s].w[2] = (uint64_t)hi; s2[s].w[3] = (uint64_t)(hi >> 64);
  }
  __float128 acc = 0, I = 0;
  for (uint64_t s = 0; s < ns; s++) {
    double c = 0.0;
    if (s1[s] != 0) {
      /* n S2 - S1^2 with n < 2^36 and S2 < 2^132: compute n * S2 limb by limb */
      u256 nS2 = u256_mul_u64(s2[s], cnt[s]);
      u256 d = u256_sub(nS2, u256_mul128(s1[s], s1[s]));
      c = sqrt(u256_to_double(d)) / (double)s1[s];
    }
    if (cov) cov[s] = c;
    const oracle_stratum* o = &R->strata[s];
    __float128 W = (__float128)(((u128)o->instr_sum_hi << 64) | o->instr_sum_lo);
    acc += W * c;
    I += W;
  }
  if (weighted) *weighted = ns ? (double)(acc / I) : 0.0;
  free(cnt); free(s1); free(s2);
  return OR_OK;
}

/* ------------------------------------------------------------------------------------------
 * NEXT-3: the exact minimum number of strata ("(1) minimises the number of strata such
 * that (2) the CoV of each stratum is below theta"; reading A28).  Per kernel, over its distinct
 * instruction counts v_1 < ... < v_m with multiplicities c_1..c_m, a stratum is a run of
 * consecutive distinct values; f(0) = 0 and
 *     f(j) = min { f(i) + 1 : 0 <= i < j, CoV(v_{i+1..j}) < theta }      (O3's exact test),
 * which always has the candidate i = j - 1 (one value: CoV 0).  The optimum is f(m); the
 * canonical optimal partition takes, at every step of the backtrack from j = m, the SMALLEST
 * i attaining f(j) - 1, and the cuts reported are the lowest value of every stratum but the
 * first, ascending.  A kernel that is one valid stratum (Tier-1/2) has f(m) = 1 and no cuts; a
 * kernel with more than max_distinct distinct values that is not is skipped (UINT32_MAX).
 * counts[K]; cuts (nullable) receives the cuts of kernels 0..K-1 in order.
 * ------------------------------------------------------------------------------------------ */
static int cmp_u64(const void* a, const void* b) {
  uint64_t x = *(const uint64_t*)a, y = *(const uint64_t*)b;
  return x < y ? -1 : x > y;
}

int oracle_min_strata(uint64_t n, uint32_t K, const uint32_t* kid, const uint64_t* x, uint32_t p,
                      uint32_t q, uint64_t max_distinct, uint32_t* counts, uint64_t* cuts,
                      uint64_t cuts_cap, uint64_t* n_cuts) {
  uint64_t total_cuts = 0;
  uint64_t* vals = (uint64_t*)malloc((n ? n : 1) * sizeof(uint64_t));
  if (!vals) return OR_ENOMEM;
  for (uint32_t k = 0; k < K; k++) {
    /* O1: the kernel's instruction counts, sorted */
    uint64_t nk = 0;
    for (uint64_t i = 0; i < n; i++) if (kid[i] == k) vals[nk++] = x[i];
    counts[k] = 0;
    if (!nk) continue;
    qsort(vals, nk, sizeof(uint64_t), cmp_u64);
    /* distinct values and their multiplicities; prefix sums N, S1, S2 over them */
    uint64_t m = 0;
    uint64_t* v = (uint64_t*)malloc(nk * sizeof(uint64_t));
    uint64_t* c = (uint64_t*)malloc(nk * sizeof(uint64_t));
    for (uint64_t i = 0; i < nk; i++) {
      if (i == 0 || vals[i] != vals[i - 1]) { v[m] = vals[i]; c[m] = 0; m++; }
      c[m - 1]++;
    }
    uint64_t* N = (uint64_t*)malloc((m + 1) * sizeof(uint64_t));
    u128* S1 = (u128*)malloc((m + 1) * sizeof(u128));
    u128* S2 = (u128*)malloc((m + 1) * sizeof(u128));
    N[0] = 0; S1[0] = 0; S2[0] = 0;
    for (uint64_t i = 0; i < m; i++) {
      N[i + 1] = N[i] + c[i];
      S1[i + 1] = S1[i] + (u128)c[i] * v[i];
      S2[i + 1] = S2[i] + (u128)c[i] * v[i] * v[i];
    }
    uint32_t best = 0;
    uint32_t* f = NULL;
    uint64_t* arg = NULL;
    if (cov_below(N[m], S1[m], S2[m], p, q)) {
      best = 1;                                   /* the whole kernel is one valid stratum */
    } else if (m > max_distinct) {
      best = UINT32_MAX;                          /* skipped */
    } else {
      f = (uint32_t*)malloc((m + 1) * sizeof(uint32_t));
      arg = (uint64_t*)malloc((m + 1) * sizeof(uint64_t));
      f[0] = 0;
      for (uint64_t j = 1; j <= m; j++) {
        f[j] = UINT32_MAX;
        for (uint64_t i = 0; i < j; i++) {
          if (f[i] + 1 < f[j] &&
              cov_below(N[j] - N[i], S1[j] - S1[i], S2[j] - S2[i], p, q)) {
            f[j] = f[i] + 1;
            arg[j] = i;                           /* strict < keeps the smallest i */
          }
        }
      }
      best = f[m];
      /* backtrack: the cuts are v at the start index of every stratum but the first */
      uint64_t nc = best - 1;
      if (cuts && total_cuts + nc <= cuts_cap) {
        uint64_t j = m, w = total_cuts + nc;
        while (j > 0) {
          uint64_t i = arg[j];
          if (i > 0) cuts[--w] = v[i];
          j = i;
        }
      }
      total_cuts += nc;
    }
    counts[k] = best;
    free(f); free(arg); free(N); free(S1); free(S2); free(v); free(c);
  }
  free(vals);
  if (n_cuts) *n_cuts = total_cuts;
  if (cuts && total_cuts > cuts_cap) return OR_ERANGE;
  return OR_OK;
}

/* accessors */
uint64_t oracle_strata_count(const oracle_result* R) { return R->n_strata; }
void oracle_strata_copy(const oracle_result* R, oracle_stratum* dst) {
  memcpy(dst, R->strata, sizeof(oracle_stratum) * R->n_strata);
}
void oracle_sid_copy(const oracle_result* R, uint32_t* dst) { memcpy(dst, R->sid, 4 * R->n); }
uint64_t oracle_segment_count(const oracle_result* R) { return R->n_segs; }
int oracle_segment_get(const oracle_result* R, uint64_t i, uint32_t* meta4, uint64_t* meta3,
                       double* h, uint64_t* d_lo, uint64_t* d_hi, uint64_t* cuts) {
  if (i >= R->n_segs) return OR_EINVAL;
  const oracle_segment* s = &R->segs[i];
  meta4[0] = s->kernel_id; meta4[1] = s->round; meta4[2] = s->split_kind; meta4[3] = s->n_cuts;
  meta3[0] = s->lo; meta3[1] = s->hi; meta3[2] = s->count;
  *h = s->bandwidth;
  if (d_lo) memcpy(d_lo, s->d_lo, 8 * R->G);
  if (d_hi) memcpy(d_hi, s->d_hi, 8 * R->G);
  if (cuts) memcpy(cuts, s->cuts, 8 * s->n_cuts);
  return OR_OK;
}
uint32_t oracle_rounds(const oracle_result* R) { return R->rounds; }
void oracle_totals(const oracle_result* R, uint64_t* out4) {
  out4[0] = (uint64_t)R->total_instr; out4[1] = (uint64_t)(R->total_instr >> 64);
  out4[2] = (uint64_t)R->c_meas; out4[3] = (uint64_t)(R->c_meas >> 64);
}
int oracle_sizeof_stratum(void) { return (int)sizeof(oracle_stratum); }
