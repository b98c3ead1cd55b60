/*
 * gen/gen_host.c -- host side of the synthetic trace generator: per-kernel tables from a seed,
 * and a multi-threaded host fill of a slice [first, first+n) of the trace.
 * Holds none of the method's arithmetic (see sieve_gen.h).
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>
#include "sieve_gen.h"

typedef struct {
  uint64_t seed, n_total;
  uint32_t K, order, homogeneous, alt_cta_pct;
  uint32_t t1_pct, t2_pct, t3_pct;        /* target shares of invocations per class */
  uint32_t t1_kernels, t2_kernels, t3_kernels; /* if nonzero: exact kernel counts per class */
  uint32_t m_min, m_max;                  /* Tier-3 modes */
  uint32_t phase_len_min, phase_len_max, n_phases, rep_min, rep_max;
} sgen_params;

typedef struct {
  sgen_tables T;
  uint64_t* zipf_cum;
  uint32_t* seq;
  uint64_t* blk_start;
  uint32_t* blk_seq_off;
  uint32_t* blk_len;
  sgen_kernel* kern;
  uint64_t seq_len;
} sgen_handle;

static double u01(uint64_t seed, uint64_t s, uint64_t i) {
  return (double)(sgen_hash(seed, s, i) >> 11) * (1.0 / 9007199254740992.0);
}

static const uint32_t CTAS[5] = {64, 128, 256, 512, 1024};

int sgen_build(const sgen_params* p, sgen_handle** out) {
  uint32_t K = p->K;
  if (K == 0 || p->m_max > SGEN_MAX_MODES || p->m_min < 1 || p->m_min > p->m_max) return -1;
  sgen_handle* H = (sgen_handle*)calloc(1, sizeof(sgen_handle));
  H->kern = (sgen_kernel*)calloc(K, sizeof(sgen_kernel));
  H->zipf_cum = (uint64_t*)malloc(sizeof(uint64_t) * K);
  uint64_t seed = p->seed;

  /* Zipf(1.0) weights over a seeded permutation of kernel ids */
  uint32_t* perm = (uint32_t*)malloc(sizeof(uint32_t) * K);
  for (uint32_t k = 0; k < K; k++) perm[k] = k;
  for (uint32_t k = K - 1; k > 0; k--) {
    uint32_t j = (uint32_t)(sgen_hash(seed, 100, k) % (k + 1));
    uint32_t t = perm[k]; perm[k] = perm[j]; perm[j] = t;
  }
  uint64_t* w = (uint64_t*)malloc(sizeof(uint64_t) * K);
  for (uint32_t r = 0; r < K; r++) w[perm[r]] = (uint64_t)(4294967296.0 / (double)(r + 1)) + 1;
  uint64_t acc = 0;
  for (uint32_t k = 0; k < K; k++) { acc += w[k]; H->zipf_cum[k] = acc; }

  /* class assignment: greedy by descending weight toward the target invocation shares,
     or exact kernel counts if given */
  uint32_t* cls = (uint32_t*)calloc(K, sizeof(uint32_t));
  if (p->t1_kernels + p->t2_kernels + p->t3_kernels > 0) {
    uint32_t want[4] = {0, p->t1_kernels, p->t2_kernels, p->t3_kernels};
    uint32_t c = 1;
    for (uint32_t r = 0; r < K; r++) {
      /* round-robin over classes that still need kernels, in rank order */
      for (int tries = 0; tries < 3; tries++) {
        if (want[c] > 0) break;
        c = c % 3 + 1;
      }
      cls[perm[r]] = want[c] > 0 ? c : 3;
      if (want[c] > 0) want[c]--;
      c = c % 3 + 1;
    }
  } else {
    double tgt[4] = {0, p->t1_pct / 100.0, p->t2_pct / 100.0, p->t3_pct / 100.0};
    double got[4] = {0, 0, 0, 0};
    double tot = (double)acc;
    for (uint32_t r = 0; r < K; r++) {
      uint32_t k = perm[r];
      int best = 1; double def = -1e300;
      for (int c = 1; c <= 3; c++) {
        double d = tgt[c] - got[c];
        if (d > def) { def = d; best = c; }
      }
      cls[k] = (uint32_t)best;
      got[best] += (double)w[k] / tot;
    }
  }

  for (uint32_t k = 0; k < K; k++) {
    sgen_kernel* G = &H->kern[k];
    G->cls = cls[k];
    G->a_k = 1 + (uint32_t)(sgen_hash(seed, 101, k) % 8);
    double base = floor(pow(10.0, 4.0 + 5.0 * u01(seed, 102, k)));
    uint32_t M = 1;
    if (cls[k] == 3) M = p->m_min + (uint32_t)(sgen_hash(seed, 103, k) % (p->m_max - p->m_min + 1));
    G->n_modes = M;
    uint32_t wc = 0;
    for (uint32_t m = 0; m < M; m++) {
      uint64_t cm = (uint64_t)base;
      uint64_t sg = 0;
      if (cls[k] == 2) {
        double cov = 0.01 + 0.14 * u01(seed, 104, k);
        sg = (uint64_t)floor(base * cov);
      } else if (cls[k] == 3) {
        double c = base * pow(2.0, 10.0 * u01(seed, 105, (uint64_t)k * 64 + m));
        if (c > 1.5e13) c = 1.5e13;
        cm = (uint64_t)floor(c);
        double cov = 0.002 + 0.028 * u01(seed, 106, (uint64_t)k * 64 + m);
        sg = (uint64_t)floor(c * cov);
      }
      G->centre[m] = cm;
      G->sigma[m] = sg;
      wc += 1 + (uint32_t)(sgen_hash(seed, 107, (uint64_t)k * 64 + m) % 100);
      G->wcum[m] = wc;
      uint32_t ci = (uint32_t)(sgen_hash(seed, 108, (uint64_t)k * 64 + m) % 5);
      G->cta[m] = CTAS[ci];
      G->cta_alt[m] = CTAS[(ci + 1 + sgen_hash(seed, 109, (uint64_t)k * 64 + m) % 4) % 5];
      G->cpi_q8[m] = 64 + (uint32_t)(sgen_hash(seed, 110, (uint64_t)k * 64 + m) % 1985);
    }
  }

  /* phase schedule */
  if (p->order == 1) {
    uint32_t P = p->n_phases;
    uint32_t* plen = (uint32_t*)malloc(sizeof(uint32_t) * P);
    uint32_t* poff = (uint32_t*)malloc(sizeof(uint32_t) * P);
    uint64_t tot = 0;
    for (uint32_t q = 0; q < P; q++) {
      plen[q] = p->phase_len_min +
                (uint32_t)(sgen_hash(seed, 120, q) % (p->phase_len_max - p->phase_len_min + 1));
      poff[q] = (uint32_t)tot;
      tot += plen[q];
    }
    H->seq = (uint32_t*)malloc(sizeof(uint32_t) * tot);
    H->seq_len = tot;
    uint64_t zt = H->zipf_cum[K - 1];
    for (uint32_t q = 0; q < P; q++)
      for (uint32_t j = 0; j < plen[q]; j++) {
        uint64_t u = sgen_hash(seed, 121, ((uint64_t)q << 32) | j) % zt;
        uint32_t lo = 0, hi = K - 1;
        while (lo < hi) { uint32_t mid = (lo + hi) >> 1; if (H->zipf_cum[mid] > u) hi = mid; else lo = mid + 1; }
        H->seq[poff[q] + j] = lo;
      }
    /* blocks: phase q = hash-chosen, repeated rep times, until n_total is covered */
    uint64_t cap = 1024, nb = 0, pos = 0;
    H->blk_start = (uint64_t*)malloc(sizeof(uint64_t) * (cap + 1));
    H->blk_seq_off = (uint32_t*)malloc(sizeof(uint32_t) * cap);
    H->blk_len = (uint32_t*)malloc(sizeof(uint32_t) * cap);
    while (pos < p->n_total || nb == 0) {
      if (nb == cap) {
        cap *= 2;
        H->blk_start = (uint64_t*)realloc(H->blk_start, sizeof(uint64_t) * (cap + 1));
        H->blk_seq_off = (uint32_t*)realloc(H->blk_seq_off, sizeof(uint32_t) * cap);
        H->blk_len = (uint32_t*)realloc(H->blk_len, sizeof(uint32_t) * cap);
      }
      uint32_t q = (uint32_t)(sgen_hash(seed, 122, nb) % P);
      uint32_t rep = p->rep_min + (uint32_t)(sgen_hash(seed, 123, nb) % (p->rep_max - p->rep_min + 1));
      H->blk_start[nb] = pos;
      H->blk_seq_off[nb] = poff[q];
      H->blk_len[nb] = plen[q];
      pos += (uint64_t)plen[q] * rep;
      nb++;
    }
    H->blk_start[nb] = pos;
    H->T.n_blk = nb;
    free(plen); free(poff);
  }
  H->T.seed = seed; H->T.K = K; H->T.order = p->order; H->T.homogeneous = p->homogeneous;
  H->T.alt_cta_pct = p->alt_cta_pct;
  H->T.zipf_cum = H->zipf_cum; H->T.seq = H->seq; H->T.blk_start = H->blk_start;
  H->T.blk_seq_off = H->blk_seq_off; H->T.blk_len = H->blk_len; H->T.kern = H->kern;
  free(perm); free(w); free(cls);
  *out = H;
  return 0;
}

void sgen_free(sgen_handle* H) {
  if (!H) return;
  free(H->kern); free(H->zipf_cum); free(H->seq); free(H->blk_start); free(H->blk_seq_off);
  free(H->blk_len); free(H);
}

/* fill rows [first, first+n) of the trace; any of the outputs may be NULL */
void sgen_fill(const sgen_handle* H, uint64_t first, uint64_t n, uint32_t* kid, uint64_t* x,
               uint32_t* cta, uint64_t* y) {
#pragma omp parallel for schedule(static)
  for (int64_t j = 0; j < (int64_t)n; j++) {
    uint32_t k, c; uint64_t xv, yv;
    sgen_row(&H->T, first + (uint64_t)j, &k, &xv, &c, &yv);
    if (kid) kid[j] = k;
    if (x) x[j] = xv;
    if (cta) cta[j] = c;
    if (y) y[j] = yv;
  }
}

/* table access for a device-side fill */
const sgen_tables* sgen_tables_of(const sgen_handle* H) { return &H->T; }
uint64_t sgen_seq_len(const sgen_handle* H) { return H->seq_len; }
uint32_t sgen_kernel_class(const sgen_handle* H, uint32_t k) { return H->kern[k].cls; }
int sgen_sizeof_kernel(void) { return (int)sizeof(sgen_kernel); }
