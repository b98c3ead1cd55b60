/*
 * gen/sieve_gen.h -- seeded, counter-based synthetic trace generator (test / bench input).
 *
 * This module holds NONE of the method's arithmetic: it only produces input rows
 * (kernel id, instruction count, CTA size, cycles) as a pure integer function of
 * (seed, global invocation index) and small per-kernel host tables.  Both the CPU oracle
 * (via tests) and the CUDA path (via tests / bench.py) consume its output; it is the only
 * module the two sides share, as allowed by the task statement.
 *
 * The recipe follows SURVEY.md 8(d): Zipf(1.0) kernel frequencies over a
 * seeded permutation; Tier-1-shaped kernels with a constant count; Tier-2-shaped kernels with
 * Irwin-Hall-12 integer noise of CoV 1-15%; Tier-3-shaped kernels with M modes whose centres
 * are log-uniform over 10 octaves and within-mode noise of 0.2-3%; CTA sizes per (kernel, mode)
 * in {64..1024} with 5% hash-selected alternates; cycles y = (x * cpi_q8) >> 8 with +-0.5%
 * noise, or y = a_k * x when `homogeneous`.  Order: i.i.d. Zipf (C1) or a training-loop
 * schedule of phases of 200-600 launches repeated in blocks (C2..C5).
 *
 * Every per-invocation function is integer-only and __host__ __device__, so a device fill
 * is bit-identical to the host fill.
 */
#ifndef SIEVE_GEN_H
#define SIEVE_GEN_H
#include <stdint.h>

#if defined(__CUDACC__)
#define SGEN_HD __host__ __device__ __forceinline__
#else
#define SGEN_HD static inline
#endif

#define SGEN_MAX_MODES 24

typedef struct {
  /* per kernel */
  uint32_t cls;                     /* 1, 2, 3 = intended tier shape */
  uint32_t n_modes;                 /* 1 for cls 1/2 */
  uint32_t a_k;                     /* homogeneous cycles factor */
  uint32_t pad;
  uint64_t centre[SGEN_MAX_MODES];  /* instruction-count centre per mode */
  uint64_t sigma[SGEN_MAX_MODES];   /* integer noise std per mode (0 for cls 1) */
  uint32_t wcum[SGEN_MAX_MODES];    /* cumulative mode weights (last = total) */
  uint32_t cta[SGEN_MAX_MODES];     /* dominant CTA size per mode */
  uint32_t cta_alt[SGEN_MAX_MODES]; /* alternate CTA size per mode */
  uint32_t cpi_q8[SGEN_MAX_MODES];  /* cycles per instruction, Q8 fixed point */
} sgen_kernel;

typedef struct {
  uint64_t seed;
  uint32_t K;
  uint32_t order;        /* 0 = i.i.d. Zipf draws, 1 = phase schedule */
  uint32_t homogeneous;  /* 1: y = a_k * x exactly */
  uint32_t alt_cta_pct;  /* % of invocations with the alternate CTA size (5) */
  uint32_t pad0, pad1;
  /* Zipf sampling table (order 0): cumulative u64 weights over kernels */
  const uint64_t* zipf_cum; /* [K] */
  /* phase schedule (order 1) */
  const uint32_t* seq;       /* concatenated phase launch sequences (kernel ids) */
  const uint64_t* blk_start; /* [n_blk+1] first invocation index of each block */
  const uint32_t* blk_seq_off; /* [n_blk] offset of the block's phase in seq */
  const uint32_t* blk_len;   /* [n_blk] phase length */
  uint64_t n_blk;
  const sgen_kernel* kern;   /* [K] */
} sgen_tables;

SGEN_HD uint64_t sgen_mix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

/* independent stream s of the counter-based generator at index i */
SGEN_HD uint64_t sgen_hash(uint64_t seed, uint64_t s, uint64_t i) {
  return sgen_mix(seed ^ sgen_mix(s * 0xD1B54A32D192ED03ull + sgen_mix(i)));
}

/* Irwin-Hall-12 integer normal: sum of 12 uniform 16-bit values, centred; std 65536 */
SGEN_HD int64_t sgen_ih12(uint64_t seed, uint64_t s, uint64_t i) {
  int64_t acc = 0;
  for (int w = 0; w < 3; w++) {
    uint64_t h = sgen_hash(seed, s * 4 + (uint64_t)w, i);
    acc += (int64_t)(h & 0xFFFF) + (int64_t)((h >> 16) & 0xFFFF) + (int64_t)((h >> 32) & 0xFFFF) +
           (int64_t)((h >> 48) & 0xFFFF);
  }
  return acc - 12 * 32768;
}

SGEN_HD uint32_t sgen_kernel_of(const sgen_tables* T, uint64_t i) {
  if (T->order == 0) {
    uint64_t tot = T->zipf_cum[T->K - 1];
    uint64_t u = sgen_hash(T->seed, 1, i) % tot;
    uint32_t lo = 0, hi = T->K - 1; /* first k with cum[k] > u */
    while (lo < hi) {
      uint32_t mid = (lo + hi) >> 1;
      if (T->zipf_cum[mid] > u) hi = mid; else lo = mid + 1;
    }
    return lo;
  }
  /* phase schedule: find block b with blk_start[b] <= i < blk_start[b+1] */
  uint64_t lo = 0, hi = T->n_blk - 1;
  while (lo < hi) {
    uint64_t mid = (lo + hi + 1) >> 1;
    if (T->blk_start[mid] <= i) lo = mid; else hi = mid - 1;
  }
  uint64_t off = i - T->blk_start[lo];
  return T->seq[T->blk_seq_off[lo] + (uint32_t)(off % T->blk_len[lo])];
}

/* one row of the trace at global index i */
SGEN_HD void sgen_row(const sgen_tables* T, uint64_t i, uint32_t* kid, uint64_t* x,
                      uint32_t* cta, uint64_t* y) {
  uint32_t k = sgen_kernel_of(T, i);
  const sgen_kernel* K = &T->kern[k];
  uint32_t m = 0;
  if (K->n_modes > 1) {
    uint32_t u = (uint32_t)(sgen_hash(T->seed, 2, i) % K->wcum[K->n_modes - 1]);
    while (K->wcum[m] <= u) m++;
  }
  int64_t v = (int64_t)K->centre[m];
  if (K->sigma[m]) {
    int64_t s = sgen_ih12(T->seed, 3, i);
    v += (s * (int64_t)K->sigma[m]) >> 16;
  }
  if (v < 1) v = 1;
  if (v > (int64_t)((1ull << 44) - 1)) v = (int64_t)((1ull << 44) - 1);
  uint64_t xv = (uint64_t)v;
  uint32_t c = K->cta[m];
  if (sgen_hash(T->seed, 4, i) % 100 < T->alt_cta_pct) c = K->cta_alt[m];
  uint64_t yv;
  if (T->homogeneous) {
    yv = (uint64_t)K->a_k * xv;
  } else {
    uint64_t base = (xv * (uint64_t)K->cpi_q8[m]) >> 8;
    int64_t jit = (int64_t)(sgen_hash(T->seed, 5, i) % 1001) - 500; /* +-0.5% */
    int64_t yy = (int64_t)base + ((int64_t)base * jit) / 100000;
    yv = yy < 1 ? 1 : (uint64_t)yy;
  }
  *kid = k; *x = xv; *cta = c; *y = yv;
}

#endif
