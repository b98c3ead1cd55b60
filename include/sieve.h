/*
 * include/sieve.h -- C-ABI of the B200-native Sieve stratification library (libsieve.so).
 *
 * Sieve (Naderan-Tahan, SeyyedAghaei, Eeckhout, ISPASS'23; /root/reference/PAPER.md, cited
 * P:NN) samples a GPU workload from its profile: "a big table with as many rows as there are
 * kernel invocations ... (kernel name, kernel invocation ID, and instruction count)" (P:59,
 * P:65).  The back-end groups invocations per kernel, tiers kernels by the
 * coefficient of variation of their instruction counts, splits high-CoV kernels
 * into strata with a kernel density estimate, picks one representative invocation per
 * stratum with an instruction-count weight, and predicts application cycles from
 * the representatives' IPC by a weighted harmonic mean.
 *
 * Every fully specified reading of an under-specified step is listed in DESIGN.md section 3
 * (A1..A24, same numbering as SURVEY.md 8(c)); the CPU oracle (oracle/) implements the same
 * readings independently, and integer outputs of this library are bit-identical to it.
 *
 * Conventions
 *   - Every call returns an int status: SIEVE_OK (0) or a negative SIEVE_E* code.  No C++
 *     exception crosses the ABI.  sieve_last_error() returns thread-local detail text.
 *   - Pointers are plain host or device pointers as documented per argument; sizes are
 *     element counts unless named *_bytes.  No framework types appear in any signature.
 *   - All device work runs on the stream given to sieve_ctx_create; every call is
 *     synchronous on return (results are complete and host outputs written).
 *   - With world > 1, sieve_stratify and sieve_predict are COLLECTIVE: every rank calls them
 *     in the same order; all ranks return identical strata (replicated decisions over exact,
 *     order-independent integer reductions, so results are byte-identical for any world size).
 */
#ifndef SIEVE_H
#define SIEVE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes ---------------------------------------------------------------------- */
enum {
  SIEVE_OK = 0,
  SIEVE_EINVAL = -1, /* null / foreign handle, theta_num or theta_den = 0, G < 3 or > 65536,
                        kernel id >= num_kernels, bad flag combination */
  SIEVE_ERANGE = -2, /* instruction count 0 or >= 2^44 (A21), n_local >= 2^32,
                        num_kernels == 0 or > 65536 */
  SIEVE_ENOMEM = -3, /* device or host allocation failed */
  SIEVE_ECUDA = -4,  /* CUDA runtime error (detail in sieve_last_error) */
  SIEVE_ENCCL = -5,  /* NCCL error or NCCL library not loadable */
  SIEVE_EDOM = -6,   /* sieve_predict without any cycle source for the representatives */
  SIEVE_ELIMIT = -7, /* the Tier-3 refinement needed more than max_rounds rounds (A15) */
  SIEVE_ESTATE = -8  /* call not valid in this state (e.g. debug data not kept) */
};

/* memory-kind flags for sieve_load_trace */
#define SIEVE_MEM_HOST 0u   /* columns are host pointers: copied to the device (H2D) */
#define SIEVE_MEM_DEVICE 1u /* columns are device pointers on the ctx's device: copied D2D */
#define SIEVE_ADOPT 2u      /* with SIEVE_MEM_DEVICE: borrow the caller's buffers, no copy; the
                               caller keeps them alive and unchanged until sieve_trace_free */
#define SIEVE_KID16 4u      /* kernel_id points to uint16_t values (K <= 65536): half the bytes
                               to copy; widened on the device.  Not with SIEVE_ADOPT */
#define SIEVE_CTA16 8u      /* cta points to uint16_t values (CTA sizes < 65536); as SIEVE_KID16 */

typedef struct sieve_ctx_s* sieve_ctx;       /* device, stream, communicator, allocator */
typedef struct sieve_trace_s* sieve_trace;   /* this rank's slice of the profile, on the device */
typedef struct sieve_strata_s* sieve_strata; /* the result; replicated on every rank */
typedef struct sieve_group_s* sieve_group;   /* in-process rank group (several ranks, one GPU) */

/* optional device allocator hook (e.g. a framework's caching allocator); stream is a
   cudaStream_t passed as void* */
typedef void* (*sieve_alloc_fn)(size_t bytes, void* stream, void* user);
typedef void (*sieve_free_fn)(void* p, void* stream, void* user);

/* ---- contexts and communicators -------------------------------------------------------- */

/* NCCL unique id for a multi-process communicator (128 bytes).  Call on rank 0 and
   broadcast the bytes to every rank by any means (e.g. torch.distributed). */
int sieve_get_unique_id(uint8_t out[128]);

/* Create a context on CUDA device `cuda_device` using stream `cuda_stream` (a cudaStream_t,
   NULL = the legacy default stream).  world > 1: ncclCommInitRank(world, *nccl_id, rank) --
   one process per GPU.  world == 1: no communicator if nccl_id is NULL; with an id, a one-rank
   NCCL communicator (the multi-rank code path on a single GPU, for testing). */
int sieve_ctx_create(int cuda_device, void* cuda_stream, int rank, int world,
                     const uint8_t* nccl_id, sieve_ctx* out);

/* In-process rank group for parity tests on ONE GPU (NCCL cannot place two ranks of one
   communicator on one device): `world` host threads each create a context with
   sieve_ctx_create_in_group and call the collective entry points concurrently; partials are
   combined by the same exact limb reductions that the NCCL path uses, through device
   memory of the shared GPU and a host barrier. */
int sieve_group_create(int world, sieve_group* out);
void sieve_group_destroy(sieve_group g);
int sieve_ctx_create_in_group(int cuda_device, void* cuda_stream, sieve_group g, int rank,
                              sieve_ctx* out);

/* Device-memory hooks (e.g. PyTorch's caching allocator); alloc and free are both set or both
   NULL (NULL restores cudaMallocAsync / cudaFreeAsync on the ctx stream).  Every buffer is
   released through the allocator that made it: a trace's owned columns keep their allocator
   until sieve_trace_free, and the context's scratch arena is returned to its allocator by this
   call (the next call grows a new arena from the new hooks).  The hooks must stay callable until
   every buffer they made is freed.  Not to be called while another call on ctx runs.
   Errors: EINVAL (bad ctx, only one hook given), ECUDA. */
int sieve_ctx_set_allocator(sieve_ctx ctx, sieve_alloc_fn alloc, sieve_free_fn free_fn, void* user);
void sieve_ctx_destroy(sieve_ctx ctx);

/* ---- the profile (extended with CTA size P:93 and cycles P:125, A20) -------- */

/* Load this rank's contiguous, chronological slice of the profile.
     n_local      rows in this slice (< 2^32); may be 0
     first_id     global invocation id of row 0 (exclusive prefix of the slice sizes); the
                  invocation ID of row j is first_id + j ("first-chronological" = the
                  smallest id, A18)
     num_kernels  K: kernel ids are dense in [0, K), 1 <= K <= 65536 ("kernel name",
                  interned by the caller); must be the same on every rank
     kernel_id    [n_local] u32
     instr        [n_local] u64 dynamic instruction count, 1 <= x < 2^44 (A21)
     cta          [n_local] u32 CTA (thread-block) size, opaque key (A16); NULL = all equal
     cycles       [n_local] u64 measured cycles; NULL = no measured cycles
     mem          SIEVE_MEM_HOST | SIEVE_MEM_DEVICE [| SIEVE_ADOPT] [| SIEVE_KID16] [| SIEVE_CTA16]
                  (the 16-bit forms change only what is copied: the trace holds u32 columns)
   Value validation (kernel id < K, 1 <= x < 2^44) happens on the device in the first pass of
   sieve_stratify, which returns SIEVE_EINVAL / SIEVE_ERANGE on a bad row.
   Return: the caller's arrays have been read in full (host or device) and may be reused; the
   widening of 16-bit columns may still run on ctx's stream, ahead of any later call's work. */
int sieve_load_trace(sieve_ctx ctx, uint64_t n_local, uint64_t first_id, uint32_t num_kernels,
                     const uint32_t* kernel_id, const uint64_t* instr, const uint32_t* cta,
                     const uint64_t* cycles, uint32_t mem, sieve_trace* out);
void sieve_trace_free(sieve_trace t);

/* Load the profile from its CSV export ("converted into a readable CSV file which serves
   as input"), parsed and interned on the GPU.  One row per invocation in
   launch order (invocation id = first_id + data-row index).  Quoted fields may contain the
   delimiter; numbers may carry thousands separators; newlines inside fields are not allowed.
   Kernel names (quote characters removed) are interned into dense ids in order of first
   appearance, identified by a 64-bit FNV-1a hash of their bytes.
     data, bytes  the CSV text: HOST (mem = SIEVE_MEM_HOST) or DEVICE (SIEVE_MEM_DEVICE)
     spec         0-based columns; col_cta / col_cycles = -1 if absent; header_lines to skip
     num_kernels  nullable: receives the number of distinct names
   SIEVE_EINVAL on a malformed row, SIEVE_ERANGE beyond 65536 names or 2^32 rows. */
typedef struct {
  int32_t col_kernel, col_instr, col_cta, col_cycles;
  uint32_t header_lines;
  char delimiter;
} sieve_csv_spec;
int sieve_load_csv(sieve_ctx ctx, const char* data, uint64_t bytes, uint32_t mem,
                   const sieve_csv_spec* spec, uint64_t first_id, sieve_trace* out,
                   uint32_t* num_kernels);
/* copy a trace's columns (n_local rows) back into HOST buffers; every pointer is nullable and a
   column the trace does not hold is left untouched.  Synchronises the context's stream. */
int sieve_trace_copy(sieve_trace t, uint32_t* kernel_id, uint64_t* instr, uint32_t* cta,
                     uint64_t* cycles, uint64_t* n_local, uint32_t* num_kernels);
/* names of a CSV-loaded trace in id order, each followed by '\n', into a HOST buffer of cap
   bytes; *needed receives the total size (call with buf = NULL to size it) */
int sieve_trace_kernel_names(sieve_trace t, char* buf, uint64_t cap, uint64_t* needed);

/* ---- stratification ------------------------------------------------------------ */
typedef struct {
  uint32_t theta_num, theta_den; /* theta = num/den, exact rational (P:85 default 0.4 = 2/5; A3) */
  uint32_t grid_points;          /* G, KDE grid points on [lo, hi] (A9), 3 <= G <= 65536; 1024 */
  uint32_t valley_shift;         /* hysteresis delta = max(1, Dmax >> shift) (A11); 10 */
  uint32_t max_rounds;           /* refinement round bound (A15); 64 */
  uint32_t keep_debug;           /* 1: keep every KDE segment for sieve_segment_get */
  double bw_scale;               /* Scott's normal-reference factor (A8); 1.06 */
} sieve_params;

void sieve_params_default(sieve_params* p);

/* Stratify the loaded profile (collective if world > 1).
     stratum_of_invocation  nullable DEVICE pointer [n_local] u32: receives the global stratum
                            index of every row of this rank's slice
     out                    the stratum table, replicated on every rank
   Strata are ordered by (kernel id, lowest instruction count) (A23). */
int sieve_stratify(sieve_trace t, const sieve_params* p, uint32_t* stratum_of_invocation,
                   sieve_strata* out);

typedef struct {
  uint32_t kernel_id;
  uint32_t tier;            /* 1, 2, 3 */
  uint32_t index_in_kernel; /* 0.. by ascending instruction counts */
  uint32_t rep_cta;         /* CTA size of the representative */
  uint64_t lo, hi;          /* smallest / largest instruction count in the stratum */
  uint64_t count;           /* invocations in the stratum */
  uint64_t instr_sum_lo, instr_sum_hi; /* W_s = sum of instruction counts, u128 */
  uint64_t rep_id;          /* global invocation id of the representative */
  uint64_t rep_instr, rep_cycles; /* x and y of the representative (y = 0 without cycles) */
  double bandwidth;         /* KDE bandwidth h of the segment whose split created this stratum;
                               0 for Tier-1/2 */
  uint32_t split_round;     /* refinement round that created it; 0 for Tier-1/2 */
  uint32_t pad;
} sieve_stratum;

int sieve_strata_count(sieve_strata s, uint64_t* n);
/* copy min(cap, count) strata to a HOST array */
int sieve_strata_copy(sieve_strata s, sieve_stratum* host_out, uint64_t cap);
/* refinement rounds used, KDE terms evaluated (diagnostics) */
/* rounds: refinement rounds; kde_terms: in-window KDE terms, i.e. (grid point j, value x) pairs
   of every round with rn(g_j - w) <= x <= rn(g_j + w), w = rn(sqrt(57) h) (0 when term counting
   is off, see sieve_ctx_set_term_count); kde_evaluated: (grid point, value) pairs the KDE kernel
   evaluated (in-window + wasted) */
int sieve_strata_stats(sieve_strata s, uint32_t* rounds, uint64_t* kde_terms,
                       uint64_t* kde_evaluated);
void sieve_strata_free(sieve_strata s);

/* ---- theta studies (Fig. 2, Fig. 10) -------------------- */

/* Stratify for `count` thresholds theta_i = theta_num[i] / theta_den[i] (host arrays) in one
   call: the per-kernel moments (pass A and its reduction) are computed once and reused; the
   Tier-3 refinement runs once, at the smallest theta, recording its tree of segments and parts,
   and every other theta takes the tree's frontier (a part is a stratum at theta where lo == hi
   or its exact CoV < theta first holds: a segment's KDE, cuts and parts depend only on its
   values), then runs tiering and the assignment.  Every table equals a separate
   sieve_stratify at that theta; kde_terms / kde_evaluated (sieve_strata_stats) are counted on
   the smallest theta's result only (the others run no KDE).  With keep_debug each theta refines
   separately.  outs[i] receives the strata for theta_i (free each with sieve_strata_free); on
   error none is returned.  Other fields of *p (grid, valley shift, ...) apply to every theta.
   Collective if world > 1. */
int sieve_stratify_sweep(sieve_trace t, const sieve_params* p, uint32_t count,
                         const uint32_t* theta_num, const uint32_t* theta_den, sieve_strata* outs);

/* Tier census (Fig. 2): for each theta_i, the number of kernels, invocations and instructions
   (u128 as lo, hi) in Tier-1/2/3, from one moments pass.  kernels, invocations: HOST
   [count][3]; instructions: nullable HOST [count][3][2].  Collective if world > 1. */
int sieve_tier_census(sieve_trace t, uint32_t count, const uint32_t* theta_num,
                      const uint32_t* theta_den, uint64_t* kernels, uint64_t* invocations,
                      uint64_t* instructions);

/* ---- debug: every KDE segment of every round (requires keep_debug = 1, else ESTATE) ---- */
typedef struct {
  uint32_t kernel_id, round, split_kind /* 1 = valley, 2 = bisect */, n_cuts;
  uint64_t lo, hi, count;
  double bandwidth;
} sieve_segment;

int sieve_segment_count(sieve_strata s, uint64_t* n);
/* density_lo/hi: nullable HOST arrays [G]: D_j as u128 = hi:lo (fixed point 2^-40, A10);
   cuts: nullable HOST array [n_cuts]: integer thresholds (x < T left, x >= T right; A12) */
int sieve_segment_get(sieve_strata s, uint64_t idx, sieve_segment* out, uint64_t* density_lo,
                      uint64_t* density_hi, uint64_t* cuts);

/* ---- prediction --------------------------------------------- */
typedef struct {
  double predicted_cycles; /* C_pred = I / IPC = sum_s W_s * y_rep / x_rep (A22) */
  double predicted_ipc;    /* IPC = 1 / sum_s w_s / IPC_s */
  double measured_cycles;  /* C_meas = sum of the trace's cycles; NaN without a cycles column */
  double error;            /* |C_pred - C_meas| / C_meas; NaN if unknown or C_meas = 0 */
  double speedup;          /* C_meas / sum_s y_rep; NaN without a cycles column */
  uint64_t total_instr_lo, total_instr_hi; /* I = sum of all instruction counts, u128 */
} sieve_prediction;

/* Predict application cycles (collective if world > 1).
     rep_cycles  nullable HOST array [n_strata]: cycles of each representative (e.g. from
                 detailed simulation); NULL = take y of the representatives from the
                 trace's cycles column (SIEVE_EDOM if the trace has none). */
int sieve_predict(sieve_strata s, sieve_trace t, const uint64_t* rep_cycles, sieve_prediction* out);

/* Predict for M cycle sources at once (Fig. 9: the same
   representatives simulated on M architectures): rep_cycles is a required HOST array
   [M][n_strata]; out is a HOST array [M].  The predicted relative speedup of architecture b
   over a is out[a].predicted_cycles / out[b].predicted_cycles.  measured_cycles / error /
   speedup refer to the trace's own cycles column (NaN without one). */
int sieve_predict_multi(sieve_strata s, sieve_trace t, uint32_t M, const uint64_t* rep_cycles,
                        sieve_prediction* out);

/* ---- measurement ------------------------------------------------------------------------ */
/* Per-phase device time of the calls made on this context, taken with CUDA events recorded on
   the context's stream around each phase (off by default; enabling resets the counters).
   `work` is the phase's algorithmic work unit count: bytes for the
   streaming passes, in-window KDE terms for SIEVE_PHASE_KDE. */
enum {
  SIEVE_PHASE_MOMENTS = 0, /* pass A: per-kernel moments */
  SIEVE_PHASE_COMPACT = 1, /* Tier-3 key compaction */
  SIEVE_PHASE_SORT = 2,    /* per round: sort of the open segments' values by (segment, grid cell) */
  SIEVE_PHASE_KDE_PLAN = 3, /* KDE planning: tile regions, item scan, work-item descriptors */
  SIEVE_PHASE_KDE = 4,     /* fixed-point KDE kernel (all rounds) */
  SIEVE_PHASE_REFINE = 5,  /* valleys + part moments (all rounds) */
  SIEVE_PHASE_ASSIGN = 6,  /* pass B: assignment + (stratum, CTA) statistics */
  SIEVE_PHASE_REPS = 7,    /* entry compaction, sort, representatives */
  SIEVE_PHASE_PREDICT = 8, /* prediction */
  SIEVE_PHASE_COUNT = 9
};
int sieve_ctx_set_timing(sieve_ctx ctx, int enable);
/* In-window KDE term counting (the KDE's algorithmic work count, sieve_strata_stats), on by
   default: one per-value grid search per round on top of the cell sort.  It changes no result;
   a timing loop over identical inputs may count once and switch it off. */
int sieve_ctx_set_term_count(sieve_ctx ctx, int enable);
int sieve_timing_get(sieve_ctx ctx, uint32_t phase, double* ms, uint64_t* calls, uint64_t* work);
/* number of kernels this process has launched through the library (all contexts) */
uint64_t sieve_kernel_launches(void);

/* ---- exact minimum number of strata (NEXT-3; reading A28) -------------- */
/* P:89 asks the Tier-3 split to "(1) minimise the number of strata such that (2) the CoV of
   each stratum is below theta".  This diagnostic computes that optimum exactly, per kernel,
   among strata that are value intervals (the only kind Sieve builds), i.e. over runs of its
   sorted distinct instruction counts: f(0) = 0, f(j) = min f(i) + 1 over the
   runs (i, j] with CoV < theta (the exact u256 test of the tiering), ties -> smallest i.
     counts      HOST [num_kernels]: 0 = no invocations, 1 = Tier-1/2 (one valid stratum), the
                 optimum for Tier-3 kernels, UINT32_MAX = skipped (more than max_distinct
                 distinct values; 0 selects 16384 -- the DP is O(m^2) per kernel)
     cuts        nullable HOST [cuts_cap]: per kernel in id order, the lowest instruction count
                 of every optimal stratum but the first, ascending (the canonical optimum: the
                 backtrack from the top takes the smallest start at every step)
     n_cuts      nullable: total number of cuts (call with cuts = NULL to size the buffer)
   SIEVE_ERANGE if cuts_cap < *n_cuts; SIEVE_ESTATE on a multi-rank context (single-rank
   diagnostic).  Synchronises the stream. */
int sieve_min_strata(sieve_trace t, uint32_t theta_num, uint32_t theta_den, uint32_t max_distinct,
                     uint32_t* counts, uint64_t* cuts, uint64_t cuts_cap, uint64_t* n_cuts);

/* ---- within-stratum cycle variability (Fig. 4; NEXT-2) ---------------------- */
/* For every stratum, the coefficient of variation of its members' cycle counts,
   cov_s = sigma_pop(y) / mean(y) = sqrt(n S2 - S1^2) / S1 from exact integer sums (0 if S1 = 0),
   and their average weighted by the strata's instruction weights W_s / I (reading A25).
     sid       DEVICE [n_local] u32: stratum_of_invocation from sieve_stratify on this trace
     cov       nullable HOST [n_strata]; weighted: nullable HOST scalar
   SIEVE_EDOM without a cycles column; SIEVE_ERANGE if a cycle count is >= 2^48.
   Collective if world > 1. */
int sieve_cycle_cov(sieve_strata s, sieve_trace t, const uint32_t* sid, double* cov, double* weighted);

/* ---- misc ----------------------------------------------------------------------------------- */
const char* sieve_last_error(void); /* thread-local; valid until the next call on this thread */
const char* sieve_version(void);

/* exact limb encoding used by every cross-rank reduction (host utility, no GPU needed):
   a u128 value is split into 32-bit limbs carried in u64 lanes so that a lane-wise u64 sum
   over up to 2^32 ranks cannot overflow; normalisation propagates the carries. */
void sieve_u128_to_limbs(uint64_t lo, uint64_t hi, uint64_t limbs[4]);
void sieve_limbs_to_u128(const uint64_t limbs[4], uint64_t* lo, uint64_t* hi);

#ifdef __cplusplus
}
#endif
#endif /* SIEVE_H */
